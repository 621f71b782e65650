timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_batched.py tests/test_gpu_attention.py -x -q -m gpu 2>&1 | tail -4
B=$PWD/build
timeout 900 python tools/tune.py --op sddmm_batched --cfg VS_SDDMM_MIX=1 --cfg VS_LIB_PATH=$B/var_noline/libvs.so --out gpurun_out/line_tune_b.json > gpurun_out/line_tune_b.log 2>&1; tail -2 gpurun_out/line_tune_b.log
timeout 900 python tools/tune.py --op sddmm --cfg VS_SDDMM_MIX=1 --cfg VS_LIB_PATH=$B/var_noline/libvs.so --out gpurun_out/line_tune.json > gpurun_out/line_tune.log 2>&1; tail -2 gpurun_out/line_tune.log
timeout 600 python bench.py --no-baselines --no-cpu --no-e2e > gpurun_out/line_bench.json 2>/dev/null; python -c "
import json;d=json.loads(open('gpurun_out/line_bench.json').read().strip().splitlines()[-1]);print(d['value'],d['ms_per_step'],{k:round(v['ms_per_step'],3) for k,v in d['kernels'].items()})"
