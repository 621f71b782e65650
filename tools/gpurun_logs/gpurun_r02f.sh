set -x
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -5 > gpurun_out/gputests.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1
timeout 600 python tools/tune.py --op sddmm_batched --cfg X=1 --out gpurun_out/tune_sddmmb.json > gpurun_out/tune_sddmmb.log 2>&1
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
cat gpurun_out/gputests.log gpurun_out/smoke.log gpurun_out/tune_sddmmb.log gpurun_out/bench.json
