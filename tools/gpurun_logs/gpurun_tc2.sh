timeout 120 ./build/umma_rate > gpurun_out/umma_rate.log 2>&1; cat gpurun_out/umma_rate.log
timeout 300 ncu --set full --import-source on -k regex:sddmm_tc -c 1 -o /tmp/tc_one python tools/one_problem.py --op sddmm --M 512 --K 2048 --N 256 --V 8 --S 0.5 > /dev/null 2>&1
python tools/ncu_summary.py full /tmp/tc_one.ncu-rep > gpurun_out/tc_one_full.md
ncu -i /tmp/tc_one.ncu-rep --page source --csv > gpurun_out/tc_one_source.csv 2>/dev/null
head -40 gpurun_out/tc_one_full.md
