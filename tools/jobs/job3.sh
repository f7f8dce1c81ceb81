# split-K v2 verification, full GPU suite (incl. config 5), racecheck, default bench, split-K trace
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "splitk" 2>&1 | tail -15 > gpurun_out/j3_splitk.log
timeout 900 compute-sanitizer --tool racecheck --print-limit 20 python tools/sanitize_cases.py > gpurun_out/j3_racecheck.log 2>&1
timeout 3000 python -m pytest tests -m gpu -q --durations=15 2>&1 | tail -40 > gpurun_out/j3_gpu_tests.log
timeout 900 python bench.py > gpurun_out/j3_bench.log 2>&1
python -m paper_conf_ipps_00020c20_b200.build -DHGEMM_TRACE --out=/tmp/libhgemm_trace.so > /dev/null 2>&1
for s in "64 4096 2048" "256 4096 2048"; do HGEMM_LIB=/tmp/libhgemm_trace.so timeout 120 python tools/trace_sk.py $s; done > gpurun_out/j3_trace_sk.log 2>&1
for f in gpurun_out/j3_*.log; do echo "== $f"; tail -n 5 $f; done
