for P in "512 2048 256 8 0.5"; do
VS_LIB_PATH=$PWD/build/var_trace/libvs.so timeout 120 python tools/tc_trace.py $P 2>&1 | cut -c1-300
done
B=$PWD/build
timeout 900 python tools/tune.py --op sddmm_batched --cfg VS_SDDMM_TC=0 --cfg VS_SDDMM_TC=1 --cfg VS_SDDMM_TC=1,VS_LIB_PATH=$B/var_s0/libvs.so --cfg VS_SDDMM_TC=1,VS_LIB_PATH=$B/var_c2/libvs.so --cfg VS_SDDMM_TC=1,VS_LIB_PATH=$B/var_c2p4/libvs.so --out gpurun_out/tc8_tune_b.json > gpurun_out/tc8_tune_b.log 2>&1; tail -6 gpurun_out/tc8_tune_b.log
