for P in "512 2048 256 8 0.5" "2048 512 256 2 0.98"; do
VS_LIB_PATH=$PWD/build/var_trace/libvs.so timeout 120 python tools/tc_trace.py $P 2>&1 | cut -c1-700
done
timeout 300 python -m pytest tests/test_gpu_parity.py tests/test_gpu_batched.py -x -q -m gpu -k sddmm 2>&1 | tail -3
timeout 600 python tools/tune.py --op sddmm_batched --cfg VS_SDDMM_TC=0 --cfg VS_SDDMM_TC=1 --out gpurun_out/tc4_tune_b.json > gpurun_out/tc4_tune_b.log 2>&1; tail -3 gpurun_out/tc4_tune_b.log
timeout 600 python tools/tune.py --op sddmm --cfg VS_SDDMM_TC=0 --cfg VS_SDDMM_TC=1 --out gpurun_out/tc4_tune.json > gpurun_out/tc4_tune.log 2>&1; tail -3 gpurun_out/tc4_tune.log
