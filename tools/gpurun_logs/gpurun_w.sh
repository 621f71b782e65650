timeout 900 python bench.py --workload c5 --steps 3 --warmup 3 > gpurun_out/w_c5.json 2>gpurun_out/w_c5.err; echo c5 rc=$?; tail -c 2500 gpurun_out/w_c5.json; tail -3 gpurun_out/w_c5.err
timeout 600 python bench.py --workload attention > gpurun_out/w_attn.json 2>gpurun_out/w_attn.err; echo attn rc=$?; tail -c 1200 gpurun_out/w_attn.json
timeout 600 python bench.py --workload attention_l8192_k64_s0.95 > gpurun_out/w_attn2.json 2>gpurun_out/w_attn2.err; echo attn2 rc=$?; tail -c 600 gpurun_out/w_attn2.json
