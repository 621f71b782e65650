set -x
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -5 > gpurun_out/gputests.log
timeout 900 python bench.py --workload c5 --steps 3 --warmup 3 > gpurun_out/bench_c5.json 2> gpurun_out/bench_c5.err
bash tools/profile_round.sh r02 > gpurun_out/profile.log 2>&1
cat gpurun_out/gputests.log gpurun_out/bench_c5.json; tail -3 gpurun_out/bench_c5.err; tail -5 gpurun_out/profile.log
