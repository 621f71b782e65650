B=$PWD/build
timeout 900 python tools/tune.py --op encode_batched --cfg VS_ENC_CHUNK_MB=0 --cfg VS_LIB_PATH=$B/var_e6/libvs.so --cfg VS_LIB_PATH=$B/var_e8/libvs.so --cfg VS_LIB_PATH=$B/var_e12/libvs.so --out gpurun_out/enc3_tune_b.json > gpurun_out/enc3_tune_b.log 2>&1; tail -4 gpurun_out/enc3_tune_b.log
