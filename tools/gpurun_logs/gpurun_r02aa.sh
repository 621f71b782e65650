#!/bin/bash
# r02aa: SDDMM unpredicated-load instantiation (K == 64 / K % 128 == 0) -- SDDMM suites, A/B vs VS_SDDMM_FAST=0
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_batched.py tests/test_gpu_coverage.py tests/test_gpu_dense.py tests/test_gpu_attention.py -q -x > gpurun_out/r02aa_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r02aa_tests.log
A="--no-cpu --no-e2e --steps 20"
for v in default nofast default nofast; do
  if [ $v = default ]; then L=paper_conf_sc_chenqldx21_b200/libvs.so; else L=build/variants/libvs_$v.so; fi
  VS_LIB_PATH=$L timeout 600 python bench.py $A --detail gpurun_out/r02aa_detail_$v.json > gpurun_out/r02aa_$v.json 2>&1
  python -c "import json;d=json.loads(open('gpurun_out/r02aa_$v.json').read().strip().splitlines()[-1]);print('$v', round(d['ms_per_step'],4), {k:round(x['ms_per_step'],4) for k,x in d['kernels'].items()}, {k:v['sddmm_vs_h'] for k,v in d['speedup_vs_cublas_hgemm']['per_cell_geomean'].items()})" >> gpurun_out/r02aa_summary.txt
done
tail -2 gpurun_out/r02aa_tests.log >> gpurun_out/r02aa_summary.txt
cat gpurun_out/r02aa_summary.txt
