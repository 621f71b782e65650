#!/bin/bash
# r02m: SDDMM K=256 body with A rows in shared memory (one round trip per chunk) A/B
A="--no-cpu --no-e2e --no-baselines --steps 20"
for v in nok256 k256m5 k256m4 nok256 k256m5; do
  VS_LIB_PATH=build/variants/libvs_$v.so timeout 300 python bench.py $A > gpurun_out/r02m_$v.json 2>&1
  python -c "import json;d=json.loads(open('gpurun_out/r02m_$v.json').read().strip().splitlines()[-1]);print('$v', round(d['ms_per_step'],4), {k:round(x['ms_per_step'],4) for k,x in d['kernels'].items()})" >> gpurun_out/r02m_summary.txt
done
for v in k256m5 k256m4; do
VS_LIB_PATH=build/variants/libvs_$v.so timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_batched.py tests/test_gpu_coverage.py tests/test_gpu_dense.py tests/test_gpu_attention.py -q -x -k "sddmm or attention or batched" > gpurun_out/r02m_tests_$v.log 2>&1
echo "$v $(tail -1 gpurun_out/r02m_tests_$v.log)" >> gpurun_out/r02m_summary.txt
done
cat gpurun_out/r02m_summary.txt
