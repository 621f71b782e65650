#!/bin/bash
# r02k: SDDMM warp/CTA layout A/B (round-robin 4x5 vs blocked 4x5 / 16x1 / 20x1) on the DLMC step
A="--no-cpu --no-e2e --no-baselines --steps 20"
for v in default pb4 pb8 pb20 default; do
  if [ $v = default ]; then L=paper_conf_sc_chenqldx21_b200/libvs.so; else L=build/variants/libvs_$v.so; fi
  VS_LIB_PATH=$L timeout 300 python bench.py $A > gpurun_out/r02k_$v.json 2>&1
  python -c "import json;d=json.loads(open('gpurun_out/r02k_$v.json').read().strip().splitlines()[-1]);print('$v', round(d['ms_per_step'],4), {k:round(x['ms_per_step'],4) for k,x in d['kernels'].items()})" >> gpurun_out/r02l_summary.txt
done
VS_LIB_PATH=build/variants/libvs_pb20.so timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_batched.py tests/test_gpu_coverage.py -q -x -k sddmm > gpurun_out/r02l_tests.log 2>&1
tail -2 gpurun_out/r02l_tests.log >> gpurun_out/r02l_summary.txt
cat gpurun_out/r02l_summary.txt
