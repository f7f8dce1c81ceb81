mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/s2_gpu_tests_a1.log 2>&1
tail -3 gpurun_out/s2_gpu_tests_a1.log
HGEMM_EXP=64 timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_large.py -x -q -k "splitk or lstm or cfg3" > gpurun_out/s2_gpu_tests_direct.log 2>&1
tail -2 gpurun_out/s2_gpu_tests_direct.log
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
