set -x
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/h2_smoke.log 2>&1; echo smoke rc=$?; tail -1 gpurun_out/h2_smoke.log
timeout 1200 python -m pytest tests -x -q -m gpu > gpurun_out/h2_pytest_gpu.log 2>&1; echo pytest rc=$?; tail -1 gpurun_out/h2_pytest_gpu.log
timeout 900 python bench.py > gpurun_out/h2_bench_full.json 2> gpurun_out/h2_bench_full.err; echo bench rc=$?
python -c "
import json;d=json.loads(open('gpurun_out/h2_bench_full.json').read().strip().splitlines()[-1]);print(d['value'],d['ms_per_step'],{k:round(v['ms_per_step'],3) for k,v in d['kernels'].items()}, d['roofline']['frac'], d['clocks'], d['config']['launch'])"
timeout 300 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/h2_bench_ref.json 2>&1; echo ref rc=$?
