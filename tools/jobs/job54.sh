# split-K: ring stages issued before the CTA barrier (1, 2, all) vs previous build (all)
mkdir -p gpurun_out
timeout 900 python -m pytest tests -q -m gpu -x -k "splitk or split_k or lstm" 2>&1 | tail -2 > gpurun_out/j54_tests.log
for rep in 1 2 3; do
  echo "PREV"; HGEMM_LIB=ab_libs/libhgemm_prev.so timeout 300 python tools/stream_sweep.py --mean --lstm
  for pre in 1 2 8; do echo "PRE $pre"; HGEMM_SK_PRE=$pre timeout 300 python tools/stream_sweep.py --mean --lstm; done
done > gpurun_out/j54_sk.log 2>&1
cat gpurun_out/j54_*.log
