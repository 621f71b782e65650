#!/bin/bash
# r04v: final default bench line (with CPU baseline + e2e) and smoke of the committed state
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r04v_smoke.log 2>&1; echo "rc=$?" >> gpurun_out/r04v_smoke.log
timeout 900 python bench.py > gpurun_out/r04v_bench.json 2> gpurun_out/r04v_bench.err
timeout 900 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/r04v_ref.json 2> gpurun_out/r04v_ref.err
tail -n 2 gpurun_out/r04v_smoke.log; grep classes gpurun_out/r04v_bench.err; tail -c 400 gpurun_out/r04v_ref.json
