timeout 600 python tools/tune.py --op encode_batched --cfg VS_ENC_L2_MB=100000 --cfg VS_ENC_L2_MB=40 --cfg VS_ENC_L2_MB=20 --cfg VS_ENC_L2_MB=70 --out gpurun_out/tune_enc.json > gpurun_out/tune_enc.log 2>&1
cat gpurun_out/tune_enc.log
