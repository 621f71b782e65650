#!/bin/bash
# r02n: pipelined e2e (default lib) + SDDMM batched grid cap A/B (3 / 4 CTAs per SM)
timeout 600 python bench.py --no-cpu --no-baselines > gpurun_out/r02n_default.json 2> gpurun_out/r02n_default.err
python -c "import json;d=json.loads(open('gpurun_out/r02n_default.json').read().strip().splitlines()[-1]);print('default', round(d['ms_per_step'],4), {k:round(x['ms_per_step'],4) for k,x in d['kernels'].items()}, 'e2e', d['e2e'])" >> gpurun_out/r02n_summary.txt
A="--no-cpu --no-e2e --no-baselines --steps 20"
for v in g3 g4; do
  VS_LIB_PATH=build/variants/libvs_$v.so timeout 300 python bench.py $A > gpurun_out/r02n_$v.json 2>&1
  python -c "import json;d=json.loads(open('gpurun_out/r02n_$v.json').read().strip().splitlines()[-1]);print('$v', round(d['ms_per_step'],4), {k:round(x['ms_per_step'],4) for k,x in d['kernels'].items()})" >> gpurun_out/r02n_summary.txt
done
cat gpurun_out/r02n_summary.txt
