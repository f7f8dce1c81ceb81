mkdir -p gpurun_out
export HGEMM_LIB=ab_libs/trace.so
echo COLD > gpurun_out/s2_trace_lstm2.log
python tools/trace_sk.py 64 4096 2048 >> gpurun_out/s2_trace_lstm2.log 2>&1
echo WARM >> gpurun_out/s2_trace_lstm2.log
python tools/trace_sk.py 64 4096 2048 --warm >> gpurun_out/s2_trace_lstm2.log 2>&1
echo COLD_NOPDL >> gpurun_out/s2_trace_lstm2.log
HGEMM_PDL=0 python tools/trace_sk.py 64 4096 2048 >> gpurun_out/s2_trace_lstm2.log 2>&1
cat gpurun_out/s2_trace_lstm2.log | grep -v "^ *[0-9]"
