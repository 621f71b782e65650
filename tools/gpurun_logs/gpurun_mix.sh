timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_batched.py tests/test_gpu_attention.py -x -q -m gpu 2>&1 | tail -2
timeout 900 python tools/tune.py --op sddmm_batched --cfg VS_SDDMM_MIX=0 --cfg VS_SDDMM_MIX=1 --out gpurun_out/mix_tune_b.json > gpurun_out/mix_tune_b.log 2>&1; tail -2 gpurun_out/mix_tune_b.log
for m in 0 1; do VS_SDDMM_MIX=$m timeout 600 python bench.py --no-baselines --no-cpu --no-e2e > gpurun_out/mix_bench_$m.json 2>/dev/null; python -c "
import json;d=json.loads(open('gpurun_out/mix_bench_$m.json').read().strip().splitlines()[-1]);print($m, d['value'],d['ms_per_step'],{k:(round(v['ms_per_step'],3),v['launches_per_step']) for k,v in d['kernels'].items()}, d['gpu_launches'])"; done
