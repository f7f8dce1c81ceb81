# split-K: receive buffer without the owner's slot (BN=128, S=2: 6 ring stages instead of 5) vs previous build
mkdir -p gpurun_out
timeout 900 python -m pytest tests -q -m gpu -x -k "splitk or split_k or lstm" 2>&1 | tail -2 > gpurun_out/j51_tests.log
for rep in 1 2 3; do
  echo "PREV"; HGEMM_LIB=ab_libs/libhgemm_prev.so timeout 300 python tools/stream_sweep.py --mean --lstm
  echo "NEW"; timeout 300 python tools/stream_sweep.py --mean --lstm
done > gpurun_out/j51_sk.log 2>&1
cat gpurun_out/j51_*.log
