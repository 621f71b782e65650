set -x
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/mb tools/microbench.cu && /tmp/mb > gpurun_out/microbench_r02.jsonl 2>&1
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -25 > gpurun_out/gputests.log
timeout 600 python tools/tune.py --op spmm --cfg VS_SPMM_CP=0 --cfg VS_SPMM_CP=3 --cfg VS_SPMM_CP=4 --cfg VS_SPMM_CP=6 --out gpurun_out/tune_spmm.json > gpurun_out/tune_spmm.log 2>&1
timeout 600 python tools/tune.py --op spmm_batched --cfg VS_SPMM_CP=0 --cfg VS_SPMM_CP=3 --cfg VS_SPMM_CP=4 --cfg VS_SPMM_CP=6 --out gpurun_out/tune_spmmb.json > gpurun_out/tune_spmmb.log 2>&1
timeout 600 python bench.py --no-baselines --no-cpu > gpurun_out/bench2.json 2> gpurun_out/bench2.err
cat gpurun_out/microbench_r02.jsonl gpurun_out/gputests.log gpurun_out/tune_spmm.log gpurun_out/tune_spmmb.log
