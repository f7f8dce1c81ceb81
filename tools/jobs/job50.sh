# split-K kernel: k-groups of 2 (3-D Ak view) vs 1; parity + LSTM timing
mkdir -p gpurun_out
timeout 900 python -m pytest tests -q -m gpu -x -k "splitk or split_k or lstm" 2>&1 | tail -3 > gpurun_out/j50_tests.log
HGEMM_SK_KG=1 timeout 900 python -m pytest tests -q -m gpu -x -k "splitk or split_k or lstm" 2>&1 | tail -2 >> gpurun_out/j50_tests.log
for rep in 1 2; do for g in 1 2; do
  echo "SK_KG $g"
  HGEMM_SK_KG=$g timeout 300 python tools/stream_sweep.py --mean --lstm
done; done > gpurun_out/j50_sk.log 2>&1
cat gpurun_out/j50_*.log
