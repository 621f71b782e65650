#!/bin/bash
# r04q: C5 step time with the dense-tile SDDMM launch (default) vs the gather-only build
for v in nopdl; do
  if [ $v = default ]; then L=paper_conf_sc_chenqldx21_b200/libvs.so; else L=build/variants/libvs_$v.so; fi
  VS_LIB_PATH=$L timeout 1500 python bench.py --workload c5 --steps 3 --warmup 3 --no-cpu --no-e2e --no-baselines > gpurun_out/r04q_$v.json 2> gpurun_out/r04q_$v.err
  python -c "import json;d=json.loads(open('gpurun_out/r04q_$v.json').read().strip().splitlines()[-1]);print('$v', round(d['value'],2), round(d['ms_per_step'],2), d['kernels'])" >> gpurun_out/r04q_summary.txt
done
cat gpurun_out/r04q_summary.txt
