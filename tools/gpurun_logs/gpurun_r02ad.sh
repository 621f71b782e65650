#!/bin/bash
# r02ac: SDDMM fast loads only for full chunks (fastfull) vs fast everywhere (default lib) vs none
VS_LIB_PATH=paper_conf_sc_chenqldx21_b200/libvs.so timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_batched.py tests/test_gpu_coverage.py -q -x -k "sddmm or batched" > gpurun_out/r02ad_tests.log 2>&1
A="--no-cpu --no-e2e --steps 20"
for v in default nofast default; do
  if [ $v = default ]; then L=paper_conf_sc_chenqldx21_b200/libvs.so; else L=build/variants/libvs_$v.so; fi
  VS_LIB_PATH=$L timeout 600 python bench.py $A > gpurun_out/r02ad_$v.json 2>&1
  python -c "import json;d=json.loads(open('gpurun_out/r02ad_$v.json').read().strip().splitlines()[-1]);print('$v', round(d['ms_per_step'],4), {k:round(x['ms_per_step'],4) for k,x in d['kernels'].items()}, {k:v['sddmm_vs_h'] for k,v in d['speedup_vs_cublas_hgemm']['per_cell_geomean'].items()})" >> gpurun_out/r02ad_summary.txt
done
tail -1 gpurun_out/r02ad_tests.log >> gpurun_out/r02ad_summary.txt
cat gpurun_out/r02ad_summary.txt
