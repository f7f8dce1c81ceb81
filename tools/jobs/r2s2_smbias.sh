mkdir -p gpurun_out
HGEMM_LIB=ab_libs/trace.so python tools/stream_sm_bias.py 64
HGEMM_LIB=ab_libs/trace.so python tools/stream_sm_bias.py 128
