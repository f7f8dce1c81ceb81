mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 900 python bench.py > gpurun_out/last_bench.log 2>&1; tail -1 gpurun_out/last_bench.log | cut -c1-300
timeout 600 python bench.py --impl reference > gpurun_out/last_ref.log 2>&1; tail -1 gpurun_out/last_ref.log | cut -c1-200
