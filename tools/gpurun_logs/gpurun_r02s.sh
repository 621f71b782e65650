#!/bin/bash
# r02s: tcgen05 gather-ring SpMM (VS_SPMM_TC=1 build) -- SpMM parity suites, then A/B vs shipped
L=build/variants/libvs_stc.so
VS_LIB_PATH=$L timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_coverage.py tests/test_gpu_batched.py tests/test_gpu_scatter.py tests/test_gpu_transpose.py tests/test_gpu_attention.py -q -x -k "spmm or scatter or batched or transpose or attention" > gpurun_out/r02s_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r02s_tests.log
A="--no-cpu --no-e2e --steps 20"
for v in stc shipped; do
  if [ $v = shipped ]; then LL=paper_conf_sc_chenqldx21_b200/libvs.so; else LL=$L; fi
  VS_LIB_PATH=$LL timeout 600 python bench.py $A --detail gpurun_out/r02s_detail_$v.json > gpurun_out/r02s_$v.json 2>&1
  python -c "import json;d=json.loads(open('gpurun_out/r02s_$v.json').read().strip().splitlines()[-1]);print('$v', round(d['ms_per_step'],4), {k:round(x['ms_per_step'],4) for k,x in d['kernels'].items()}, {k:v['spmm_vs_h'] for k,v in d['speedup_vs_cublas_hgemm']['per_cell_geomean'].items()})" >> gpurun_out/r02s_summary.txt 2>&1
done
tail -3 gpurun_out/r02s_tests.log >> gpurun_out/r02s_summary.txt
cat gpurun_out/r02s_summary.txt
