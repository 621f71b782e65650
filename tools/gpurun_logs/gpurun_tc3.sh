for P in "512 2048 256 8 0.5" "2048 512 256 2 0.98"; do
VS_LIB_PATH=$PWD/build/var_trace/libvs.so timeout 120 python tools/tc_trace.py $P > gpurun_out/tc_trace_$(echo $P|tr ' ' _).log 2>&1
cat gpurun_out/tc_trace_$(echo $P|tr ' ' _).log | cut -c1-1500
done
