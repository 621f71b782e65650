#!/bin/bash
# r04u: shipped state candidate: ring depth per launch + PDL only for dense grids <= 8192 units
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/r04u_gputest.log 2>&1; echo "rc=$?" >> gpurun_out/r04u_gputest.log
timeout 600 python bench.py --no-cpu --no-e2e > gpurun_out/r04u_bench.json 2> gpurun_out/r04u_bench.err
cp gpurun_out/bench_detail.json gpurun_out/r04u_detail.json
timeout 900 python bench.py --workload rn50_layer --no-cpu --no-e2e > gpurun_out/r04u_rn50.json 2> gpurun_out/r04u_rn50.err
timeout 1500 python bench.py --workload c5 --steps 3 --warmup 3 --no-cpu --no-e2e --no-baselines > gpurun_out/r04u_c5.json 2> gpurun_out/r04u_c5.err
tail -n 2 gpurun_out/r04u_gputest.log; grep classes gpurun_out/r04u_bench.err gpurun_out/r04u_rn50.err
python -c "import json;d=json.loads(open('gpurun_out/r04u_c5.json').read().strip().splitlines()[-1]);print('c5', round(d['value'],2), round(d['ms_per_step'],2))"
