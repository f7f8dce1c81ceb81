mkdir -p gpurun_out
export HGEMM_LIB=ab_libs/trace.so
python tools/trace_stream.py 64 4096 2048 1.0 --force > gpurun_out/s2_trace_lstm.log 2>&1
python tools/trace_stream.py 64 4096 2048 1.0 64 >> gpurun_out/s2_trace_lstm.log 2>&1
python tools/trace_sk.py 64 4096 2048 >> gpurun_out/s2_trace_lstm.log 2>&1
HGEMM_PDL=0 python tools/trace_sk.py 64 4096 2048 >> gpurun_out/s2_trace_lstm.log 2>&1
HGEMM_PDL=0 python tools/trace_stream.py 64 4096 2048 1.0 --force >> gpurun_out/s2_trace_lstm.log 2>&1
cat gpurun_out/s2_trace_lstm.log
