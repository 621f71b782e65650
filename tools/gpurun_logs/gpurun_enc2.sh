timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_batched.py -x -q -m gpu -k "encode or batched" 2>&1 | tail -2
B=$PWD/build
timeout 900 python tools/tune.py --op encode_batched --cfg VS_ENC_CHUNK_MB=0 --cfg VS_LIB_PATH=$B/var_direct/libvs.so --out gpurun_out/enc2_tune_b.json > gpurun_out/enc2_tune_b.log 2>&1; tail -3 gpurun_out/enc2_tune_b.log
