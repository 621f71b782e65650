# SDDMM grid oversubscription under the SDDMM-priority chain schedule
run() {
  env "$@" timeout 600 python bench.py --steps 20 --warmup 5 --no-baselines --no-cpu --no-e2e > gpurun_out/s_bench.json 2>/dev/null
  python -c "
import json,sys;d=json.loads(open('gpurun_out/s_bench.json').read().strip().splitlines()[-1]);print(sys.argv[1:], round(d['value'],3), round(d['ms_per_step'],4))" "$@" | tee -a gpurun_out/s_sweep.txt
}
for i in 1 2; do
run VS_SDDMM_OVERSUB=1
run VS_SDDMM_OVERSUB=2
run VS_SDDMM_OVERSUB=3
done
