# chain-schedule stream priorities (bench.py --priority)
run() {
  timeout 600 python bench.py --steps 20 --warmup 5 --no-baselines --no-cpu --no-e2e "$@" > gpurun_out/r_bench.json 2>gpurun_out/r_bench.err
  python -c "
import json,sys;d=json.loads(open('gpurun_out/r_bench.json').read().strip().splitlines()[-1]);print(sys.argv[1:], round(d['value'],3), round(d['ms_per_step'],4))" "$@" | tee -a gpurun_out/r_sweep.txt
}
for i in 1 2; do
run --priority none
run --priority first
run --priority sddmm
run --priority encode
done
tail -3 gpurun_out/r_bench.err
