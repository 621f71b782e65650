timeout 900 python -m pytest tests -x -q -m gpu > gpurun_out/tc10_pytest.log 2>&1; echo pytest rc=$?; tail -3 gpurun_out/tc10_pytest.log
timeout 600 python bench.py --no-baselines --no-cpu --no-e2e > gpurun_out/tc10_bench.json 2>/dev/null; echo bench rc=$?
python -c "
import json;d=json.loads(open('gpurun_out/tc10_bench.json').read().strip().splitlines()[-1]);print(d['value'],d['ms_per_step'],{k:round(v['ms_per_step'],3) for k,v in d['kernels'].items()})"
