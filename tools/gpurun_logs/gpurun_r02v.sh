#!/bin/bash
# r02v: single-pass encoder (fused count + look-back + compact) -- encode tests, A/B vs two-pass
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_batched.py tests/test_gpu_coverage.py tests/test_gpu_dense.py tests/test_gpu_transpose.py -q -x > gpurun_out/r02v_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r02v_tests.log
A="--no-cpu --no-e2e --no-baselines --steps 20"
for v in default enc2p default enc2p; do
  if [ $v = default ]; then L=paper_conf_sc_chenqldx21_b200/libvs.so; else L=build/variants/libvs_$v.so; fi
  VS_LIB_PATH=$L timeout 300 python bench.py $A > gpurun_out/r02v_$v.json 2>&1
  python -c "import json;d=json.loads(open('gpurun_out/r02v_$v.json').read().strip().splitlines()[-1]);print('$v', round(d['ms_per_step'],4), {k:round(x['ms_per_step'],4) for k,x in d['kernels'].items()})" >> gpurun_out/r02v_summary.txt 2>&1
done
tail -2 gpurun_out/r02v_tests.log >> gpurun_out/r02v_summary.txt
cat gpurun_out/r02v_summary.txt
