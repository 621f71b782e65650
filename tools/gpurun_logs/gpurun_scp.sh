VS_SDDMM_CP=1 timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_batched.py -x -q -m gpu -k "sddmm or batched" 2>&1 | tail -3
timeout 900 python tools/tune.py --op sddmm_batched --cfg VS_SDDMM_CP=0 --cfg VS_SDDMM_CP=1 --cfg VS_SDDMM_CP=1,VS_SDDMM_KC=1 --out gpurun_out/scp_tune_b.json > gpurun_out/scp_tune_b.log 2>&1; tail -3 gpurun_out/scp_tune_b.log
timeout 900 python tools/tune.py --op sddmm --cfg VS_SDDMM_CP=0 --cfg VS_SDDMM_CP=1 --out gpurun_out/scp_tune.json > gpurun_out/scp_tune.log 2>&1; tail -2 gpurun_out/scp_tune.log
