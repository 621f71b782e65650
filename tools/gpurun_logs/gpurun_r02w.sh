#!/bin/bash
# r02v: single-pass encoder (fused count + look-back + compact) -- encode tests, A/B vs two-pass
VS_LIB_PATH=build/variants/libvs_t4.so timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_batched.py -q -x -k encode > gpurun_out/r02w_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r02w_tests.log
A="--no-cpu --no-e2e --no-baselines --steps 20"
for v in t4 t8 t16 enc2p; do
  if [ $v = default ]; then L=paper_conf_sc_chenqldx21_b200/libvs.so; else L=build/variants/libvs_$v.so; fi
  VS_LIB_PATH=$L timeout 300 python bench.py $A > gpurun_out/r02w_$v.json 2>&1
  python -c "import json;d=json.loads(open('gpurun_out/r02w_$v.json').read().strip().splitlines()[-1]);print('$v', round(d['ms_per_step'],4), {k:round(x['ms_per_step'],4) for k,x in d['kernels'].items()})" >> gpurun_out/r02w_summary.txt 2>&1
done
tail -2 gpurun_out/r02w_tests.log >> gpurun_out/r02w_summary.txt
cat gpurun_out/r02w_summary.txt
