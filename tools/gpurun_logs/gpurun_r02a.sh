#!/bin/bash
# r02a: GPU suite after the round-2 parity additions + frozen knobs, then the default bench
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02a_smoke.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r02a_gputest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r02a_gputest.log
timeout 600 python bench.py > gpurun_out/r02a_bench.json 2> gpurun_out/r02a_bench.err
tail -3 gpurun_out/r02a_gputest.log
