B=$PWD/build
timeout 900 python tools/tune.py --op sddmm_batched --cfg VS_SDDMM_MIX=1 --cfg VS_LIB_PATH=$B/var_m4/libvs.so --cfg VS_LIB_PATH=$B/var_m6/libvs.so --out gpurun_out/m2_tune_b.json > gpurun_out/m2_tune_b.log 2>&1; tail -3 gpurun_out/m2_tune_b.log
