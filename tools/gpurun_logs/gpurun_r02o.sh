#!/bin/bash
# r02o: packed, pipelined e2e at 6 / 12 / 24 chunks
for c in 12 6 24; do
timeout 600 python bench.py --no-cpu --no-baselines --e2e-chunks $c --steps 10 > gpurun_out/r02o_e2e$c.json 2> gpurun_out/r02o_e2e$c.err
python -c "import json;d=json.loads(open('gpurun_out/r02o_e2e$c.json').read().strip().splitlines()[-1]);e=d['e2e'];print('chunks $c step', round(d['ms_per_step'],4), 'e2e', round(e['ms_per_step'],3), 'serial', round(e['serialized_ms_per_step'],3), 'value', round(e['value'],3))" >> gpurun_out/r02o_summary.txt 2>&1
done
cat gpurun_out/r02o_summary.txt; tail -3 gpurun_out/r02o_e2e12.err
