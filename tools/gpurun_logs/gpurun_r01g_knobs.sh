# re-sweep of the run-time knobs after the PDL / paired-SDDMM / encode-prefetch changes
run() {
  env "$@" timeout 600 python bench.py --steps 20 --warmup 5 --no-baselines --no-cpu --no-e2e > gpurun_out/k_bench.json 2>/dev/null
  python -c "
import json,sys;d=json.loads(open('gpurun_out/k_bench.json').read().strip().splitlines()[-1]);print(sys.argv[1:], round(d['value'],3), round(d['ms_per_step'],4), {k:round(v['ms_per_step'],4) for k,v in d['kernels'].items()})" "$@" | tee -a gpurun_out/k_sweep.txt
}
run VS_NONE=1
run VS_SPMM_CP=3
run VS_SPMM_CPNC=1
run VS_SPMM_CPNC=4
run VS_SDDMM_OVERSUB=2
run VS_SDDMM_KC=1
run VS_SPMM_PDL=0
run VS_NONE=2
