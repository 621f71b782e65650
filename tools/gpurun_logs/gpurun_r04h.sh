#!/bin/bash
# r04h: final shipped state (dense-tile SDDMM, 1 stage / 4 CTAs per SM): smoke, full GPU suite, default bench, ncu profile round
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r04h_smoke.log 2>&1; echo "rc=$?" >> gpurun_out/r04h_smoke.log
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/r04h_gputest.log 2>&1; echo "rc=$?" >> gpurun_out/r04h_gputest.log
timeout 900 python bench.py > gpurun_out/r04h_bench.json 2> gpurun_out/r04h_bench.err
cp gpurun_out/bench_detail.json gpurun_out/r04h_detail.json
bash tools/profile_round.sh r04 > gpurun_out/profile_r04.log 2>&1
tail -n 2 gpurun_out/r04h_smoke.log gpurun_out/r04h_gputest.log; grep classes gpurun_out/r04h_bench.err
