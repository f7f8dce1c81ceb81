mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "splitk or small_problems or lstm" > gpurun_out/s2_tmb_tests.log 2>&1; tail -2 gpurun_out/s2_tmb_tests.log
for v in new base; do
  if [ $v = base ]; then export HGEMM_LIB=ab_libs/base9.so; else unset HGEMM_LIB; fi
  for wl in cfg3_lstm_b64 cfg3_lstm_b256 cfg1_256_NN_f32; do
    python tools/ncu_configs.py $wl > /dev/null 2>&1
    ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/tmb_${v}_$wl.csv \
       python tools/ncu_configs.py $wl > gpurun_out/tmb_${v}_${wl}_order.txt 2>/dev/null
    echo "== $v $wl"; python tools/launch_cost_join.py gpurun_out/tmb_${v}_$wl.csv gpurun_out/tmb_${v}_${wl}_order.txt | grep -E "auto|splitk/64/2|splitk/64/4|splitk/128/2"
  done
done
unset HGEMM_LIB
HGEMM_LIB=ab_libs/trace.so python tools/trace_sk.py 64 4096 2048 | grep -v "^ *[0-9]"
HGEMM_EXP=64 timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "splitk" 2>&1 | tail -1
