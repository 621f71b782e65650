B=$PWD/build
timeout 900 python tools/tune.py --op sddmm_batched --cfg VS_SDDMM_TC=0 --cfg VS_LIB_PATH=$B/var_m5/libvs.so --cfg VS_LIB_PATH=$B/var_m6/libvs.so --cfg VS_LIB_PATH=$B/var_m8/libvs.so --cfg VS_SDDMM_KC=1 --out gpurun_out/m1_tune_b.json > gpurun_out/m1_tune_b.log 2>&1; tail -6 gpurun_out/m1_tune_b.log
