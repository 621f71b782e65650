set -x
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
bash tools/profile_round.sh r02 > gpurun_out/profile.log 2>&1
cat gpurun_out/bench.json; grep -v "^+" gpurun_out/profile.log | tail -5
