# wave barrier on by default: full GPU suite, default bench with / without it, sustained 8192 / 16384
mkdir -p gpurun_out
timeout 3000 python -m pytest tests -m gpu -q -x 2>&1 | tail -4 > gpurun_out/j18_gpu_tests.log
for r in 1 2; do
  timeout 900 python bench.py --no-cpu --no-side > gpurun_out/j18_bench_wsync1_$r.log 2>&1
  HGEMM_WSYNC=0 timeout 900 python bench.py --no-cpu --no-side > gpurun_out/j18_bench_wsync0_$r.log 2>&1
done
for rep in 1 2; do for w in 1 0; do
  HGEMM_WSYNC=$w timeout 200 python tools/sustained.py --m 8192 --warm 2 --iters 300 --order ours | sed "s/^/8192 wsync$w /"
done; done > gpurun_out/j18_sustained.log 2>&1
python - <<'PY'
import json, glob
for f in sorted(glob.glob("gpurun_out/j18_bench_*.log")):
    l = [x for x in open(f) if x.startswith("{")]
    if not l: print(f, "no line"); continue
    d = json.loads(l[-1])
    s = d["strong_32768"]
    print(f.split("/")[-1], f"value {d['value']:.1f} cublas {d['cublas']['value']:.1f} agree {d['cublas'].get('agrees_with_ours')} "
          f"clk {d['clocks'].get('sm_mhz_in_kernel_median', 0):.0f} | strong t_gemm {s.get('t_gemm_ms', 0):.2f} ms "
          f"{s.get('TFLOP/s_aggregate', 0):.1f} TF cublas {s.get('cublas_slab_TFLOP/s', 0):.1f} | e2e {d['e2e']['value']:.1f}")
PY
cat gpurun_out/j18_gpu_tests.log gpurun_out/j18_sustained.log
