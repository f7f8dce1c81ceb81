# skinny streaming A/B: k rotation, ring depth, chunk width
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for rot in 1 0; do for st in 0 4 6; do
  echo "ROT $rot STAGES $st"
  HGEMM_STREAM_ROT=$rot HGEMM_STREAM_STAGES=$st timeout 300 python tools/stream_sweep.py --skinny
done; done > gpurun_out/j38_skinny_ab.log 2>&1
cat gpurun_out/j38_skinny_ab.log
