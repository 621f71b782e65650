set -x
timeout 900 python -m pytest tests -x -q -m gpu -k "encode or batched or smoke or transpose or train" > gpurun_out/h_pytest.log 2>&1; echo pytest rc=$?; tail -2 gpurun_out/h_pytest.log
for i in 1 2; do
timeout 600 python bench.py --steps 20 --warmup 5 --no-baselines --no-cpu --no-e2e > gpurun_out/h_bench_${i}.json 2>/dev/null
python -c "
import json;d=json.loads(open('gpurun_out/h_bench_${i}.json').read().strip().splitlines()[-1]);print('PF', round(d['value'],3), round(d['ms_per_step'],4), {k:round(v['ms_per_step'],4) for k,v in d['kernels'].items()})"
done
