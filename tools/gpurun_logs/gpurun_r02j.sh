set -x
W24=$PWD/build/var_w24/libvs.so; W32=$PWD/build/var_w32/libvs.so
CFGS="--cfg VS_SPMM_CP=3 --cfg VS_SPMM_CP=2 --cfg VS_SPMM_CP=2,VS_LIB_PATH=$W24 --cfg VS_SPMM_CP=3,VS_LIB_PATH=$W24 --cfg VS_SPMM_CP=2,VS_LIB_PATH=$W32"
timeout 900 python tools/tune.py --op spmm_batched $CFGS --out gpurun_out/tune_spmmb.json > gpurun_out/tune_spmmb.log 2>&1
timeout 900 python tools/tune.py --op spmm $CFGS --out gpurun_out/tune_spmm.json > gpurun_out/tune_spmm.log 2>&1
for i in 1 2; do timeout 600 python bench.py --no-baselines --no-cpu --no-e2e > gpurun_out/bench_v$i.json 2>/dev/null; done
cat gpurun_out/tune_spmmb.log gpurun_out/tune_spmm.log
for i in 1 2; do python -c "
import json;d=json.loads(open('gpurun_out/bench_v$i.json').read().strip().splitlines()[-1]);print(d['value'],d['ms_per_step'],{k:round(v['ms_per_step'],3) for k,v in d['kernels'].items()})"; done
