# split-K: ring stage cap 8 (kg=2: all 8 k-blocks of b64 in flight) vs 6
mkdir -p gpurun_out
timeout 900 python -m pytest tests -q -m gpu -x -k "splitk or split_k or lstm" 2>&1 | tail -2 > gpurun_out/j52_tests.log
for rep in 1 2 3; do
  echo "PREV"; HGEMM_LIB=ab_libs/libhgemm_prev.so timeout 300 python tools/stream_sweep.py --mean --lstm
  echo "NEW"; timeout 300 python tools/stream_sweep.py --mean --lstm
done > gpurun_out/j52_sk.log 2>&1
cat gpurun_out/j52_*.log
