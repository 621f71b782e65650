set -x
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -25 > gpurun_out/gputests.log
timeout 900 python tools/tune.py --op sddmm --cfg VS_SDDMM_KC=2 --cfg VS_SDDMM_KC=1 --out gpurun_out/tune_sddmm.json > gpurun_out/tune_sddmm.log 2>&1
timeout 600 python tools/tune.py --op sddmm_batched --cfg VS_SDDMM_KC=2 --cfg VS_SDDMM_KC=1 --out gpurun_out/tune_sddmmb.json > gpurun_out/tune_sddmmb.log 2>&1
cat gpurun_out/gputests.log gpurun_out/tune_sddmm.log gpurun_out/tune_sddmmb.log
