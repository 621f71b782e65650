set -x
timeout 180 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k sddmm > gpurun_out/tc1_sddmm_tests.log 2>&1; echo sddmm-tests rc=$?
tail -15 gpurun_out/tc1_sddmm_tests.log
timeout 600 python -m pytest tests -x -q -m gpu > gpurun_out/tc1_pytest.log 2>&1; echo pytest rc=$?
tail -15 gpurun_out/tc1_pytest.log
timeout 600 python tools/tune.py --op sddmm_batched --cfg VS_SDDMM_TC=0 --cfg VS_SDDMM_TC=1 --out gpurun_out/tc1_tune_b.json > gpurun_out/tc1_tune_b.log 2>&1; tail -8 gpurun_out/tc1_tune_b.log
timeout 600 python tools/tune.py --op sddmm --cfg VS_SDDMM_TC=0 --cfg VS_SDDMM_TC=1 --out gpurun_out/tc1_tune.json > gpurun_out/tc1_tune.log 2>&1; tail -8 gpurun_out/tc1_tune.log
timeout 600 python bench.py --no-baselines --no-cpu --no-e2e > gpurun_out/tc1_bench.json 2>gpurun_out/tc1_bench.err; echo bench rc=$?
python -c "
import json;d=json.loads(open('gpurun_out/tc1_bench.json').read().strip().splitlines()[-1]);print(d['value'],d['ms_per_step'],{k:round(v['ms_per_step'],3) for k,v in d['kernels'].items()})"
