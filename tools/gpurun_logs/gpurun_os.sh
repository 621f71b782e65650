timeout 900 python tools/tune.py --op sddmm_batched --cfg VS_SDDMM_OVERSUB=1 --cfg VS_SDDMM_OVERSUB=2 --cfg VS_SDDMM_OVERSUB=4 --out gpurun_out/os_tune_b.json > gpurun_out/os_tune_b.log 2>&1; tail -3 gpurun_out/os_tune_b.log
for o in 1 2 4; do VS_SDDMM_OVERSUB=$o timeout 600 python bench.py --no-baselines --no-cpu --no-e2e > gpurun_out/os_bench_$o.json 2>/dev/null; python -c "
import json;d=json.loads(open('gpurun_out/os_bench_$o.json').read().strip().splitlines()[-1]);print($o, d['value'],d['ms_per_step'],{k:round(v['ms_per_step'],3) for k,v in d['kernels'].items()})"; done
