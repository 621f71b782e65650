#!/bin/bash
# r03a: re-entry baseline of the restored HEAD: smoke, full GPU suite, default bench
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r03a_smoke.log 2>&1; echo "rc=$?" >> gpurun_out/r03a_smoke.log
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/r03a_gputest.log 2>&1; echo "rc=$?" >> gpurun_out/r03a_gputest.log
timeout 900 python bench.py > gpurun_out/r03a_bench.json 2> gpurun_out/r03a_bench.err
tail -2 gpurun_out/r03a_smoke.log gpurun_out/r03a_gputest.log; tail -c 1500 gpurun_out/r03a_bench.json
