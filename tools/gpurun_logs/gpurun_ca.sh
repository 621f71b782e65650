B=$PWD/build
timeout 900 python tools/tune.py --op spmm_batched --cfg VS_SPMM_CP=2 --cfg VS_LIB_PATH=$B/var_ca/libvs.so --cfg VS_LIB_PATH=$B/var_ca_w32/libvs.so --cfg VS_LIB_PATH=$B/var_ca_w16/libvs.so --cfg VS_LIB_PATH=$B/var_ca/libvs.so,VS_SPMM_CPNC=1 --cfg VS_LIB_PATH=$B/var_ca/libvs.so,VS_SPMM_CPNC=4 --out gpurun_out/ca_tune_b.json > gpurun_out/ca_tune_b.log 2>&1; tail -7 gpurun_out/ca_tune_b.log
timeout 900 python tools/tune.py --op spmm --cfg VS_SPMM_CP=2 --cfg VS_LIB_PATH=$B/var_ca/libvs.so --out gpurun_out/ca_tune.json > gpurun_out/ca_tune.log 2>&1; tail -3 gpurun_out/ca_tune.log
