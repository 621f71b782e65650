timeout 300 python -m pytest tests/test_gpu_parity.py tests/test_gpu_batched.py tests/test_gpu_attention.py -x -q -m gpu 2>&1 | tail -3
for P in "512 2048 256 8 0.5" "2048 512 256 2 0.98"; do
VS_LIB_PATH=$PWD/build/var_trace/libvs.so timeout 120 python tools/tc_trace.py $P 2>&1 | cut -c1-500
done
B=$PWD/build
timeout 900 python tools/tune.py --op sddmm_batched --cfg VS_SDDMM_TC=0 --cfg VS_SDDMM_TC=1 --cfg VS_SDDMM_TC=1,VS_LIB_PATH=$B/var_p16/libvs.so --cfg VS_SDDMM_TC=1,VS_LIB_PATH=$B/var_p4/libvs.so --out gpurun_out/tc5_tune_b.json > gpurun_out/tc5_tune_b.log 2>&1; tail -5 gpurun_out/tc5_tune_b.log
timeout 900 python tools/tune.py --op sddmm --cfg VS_SDDMM_TC=0 --cfg VS_SDDMM_TC=1 --cfg VS_SDDMM_TC=1,VS_LIB_PATH=$B/var_p16/libvs.so --out gpurun_out/tc5_tune.json > gpurun_out/tc5_tune.log 2>&1; tail -4 gpurun_out/tc5_tune.log
