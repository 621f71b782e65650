set -x
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -25 > gpurun_out/gputests.log
CFGS="--cfg VS_SPMM_CP=0 --cfg VS_SPMM_CP=3,VS_SPMM_CPNC=1 --cfg VS_SPMM_CP=3,VS_SPMM_CPNC=2 --cfg VS_SPMM_CP=3 --cfg VS_SPMM_CP=4"
timeout 900 python tools/tune.py --op spmm $CFGS --out gpurun_out/tune_spmm.json > gpurun_out/tune_spmm.log 2>&1
timeout 600 python tools/tune.py --op spmm_batched $CFGS --out gpurun_out/tune_spmmb.json > gpurun_out/tune_spmmb.log 2>&1
cat gpurun_out/gputests.log gpurun_out/tune_spmm.log gpurun_out/tune_spmmb.log
