for s in chains phases; do timeout 600 python bench.py --no-baselines --no-cpu --schedule $s > gpurun_out/ch_bench_$s.json 2>gpurun_out/ch_bench_$s.err; echo rc=$?; python -c "
import json;d=json.loads(open('gpurun_out/ch_bench_$s.json').read().strip().splitlines()[-1]);print('$s', d['value'],d['ms_per_step'],d['alt_schedule'],d['gpu_launches'],d['e2e']['value'])"; done
