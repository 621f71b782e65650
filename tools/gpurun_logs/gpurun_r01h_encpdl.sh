set -x
timeout 900 python -m pytest tests -x -q -m gpu -k "encode or batched or smoke or transpose or train or attention" > gpurun_out/e2_pytest.log 2>&1; echo pytest rc=$?; tail -2 gpurun_out/e2_pytest.log
for i in 1 2; do
for P in 0 1; do
VS_ENC_PDL=$P timeout 600 python bench.py --steps 20 --warmup 5 --no-baselines --no-cpu --no-e2e > gpurun_out/e2_bench_${P}_${i}.json 2>/dev/null
python -c "
import json;d=json.loads(open('gpurun_out/e2_bench_${P}_${i}.json').read().strip().splitlines()[-1]);print('PAIR=$P', round(d['value'],3), round(d['ms_per_step'],4), {k:round(v['ms_per_step'],4) for k,v in d['kernels'].items()})"
done; done
