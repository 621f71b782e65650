set -x
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/g_smoke.log 2>&1; echo smoke rc=$?; tail -2 gpurun_out/g_smoke.log
timeout 1200 python -m pytest tests -x -q -m gpu > gpurun_out/g_pytest_gpu.log 2>&1; echo pytest rc=$?
tail -3 gpurun_out/g_pytest_gpu.log
timeout 900 python bench.py > gpurun_out/g_bench_full.json 2> gpurun_out/g_bench_full.err; echo bench rc=$?
python -c "
import json;d=json.loads(open('gpurun_out/g_bench_full.json').read().strip().splitlines()[-1]);print(d['value'],d['ms_per_step'],{k:round(v['ms_per_step'],3) for k,v in d['kernels'].items()}, d['roofline'], d.get('speedup_vs_cublas_hgemm',{}).get('geomean_spmm'), d.get('speedup_vs_cublas_hgemm',{}).get('geomean_sddmm'))"
timeout 300 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/g_bench_ref.json 2>&1; echo ref rc=$?
bash tools/profile_round.sh r01g > gpurun_out/g_profile.log 2>&1; echo prof rc=$?
timeout 600 compute-sanitizer --tool memcheck --error-exitcode 9 python -m pytest tests/test_gpu_batched.py -x -q -m gpu > gpurun_out/g_memcheck.log 2>&1; echo memcheck rc=$?; tail -3 gpurun_out/g_memcheck.log
