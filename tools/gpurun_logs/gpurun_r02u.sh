#!/bin/bash
# r02u: SDDMM two accumulation chains (VS_SDDMM_ACC2=1) A/B vs default; SDDMM suites on the variant
VS_LIB_PATH=build/variants/libvs_acc2.so timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_batched.py tests/test_gpu_coverage.py -q -x -k "sddmm or batched" > gpurun_out/r02u_tests.log 2>&1
A="--no-cpu --no-e2e --no-baselines --steps 20"
for v in default acc2 default acc2; do
  if [ $v = default ]; then L=paper_conf_sc_chenqldx21_b200/libvs.so; else L=build/variants/libvs_$v.so; fi
  VS_LIB_PATH=$L timeout 300 python bench.py $A > gpurun_out/r02u_$v.json 2>&1
  python -c "import json;d=json.loads(open('gpurun_out/r02u_$v.json').read().strip().splitlines()[-1]);print('$v', round(d['ms_per_step'],4), {k:round(x['ms_per_step'],4) for k,x in d['kernels'].items()})" >> gpurun_out/r02u_summary.txt
done
tail -1 gpurun_out/r02u_tests.log >> gpurun_out/r02u_summary.txt
cat gpurun_out/r02u_summary.txt
