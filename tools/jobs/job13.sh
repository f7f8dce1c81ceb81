# N > 1 code path of bench.py with two ranks sharing one GPU (gloo for the process group, CUDA IPC
# for the fused all-gather): exercises strong_32768 + the exchange legs end to end (no performance meaning)
mkdir -p gpurun_out
HGEMM_DIST_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 \
  --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 2 --steps 3 --warmup 3 --no-cpu --no-cublas \
  > gpurun_out/j13_bench_n2_gloo.log 2>&1
echo "rc=$?" >> gpurun_out/j13_bench_n2_gloo.log
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 \
  --master-port 29512 bench.py --gpus 1 --steps 3 --warmup 3 --no-cpu --no-side > gpurun_out/j13_bench_n1_torchrun.log 2>&1
echo "rc=$?" >> gpurun_out/j13_bench_n1_torchrun.log
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 --ref-budget 20 > gpurun_out/j13_reference.log 2>&1
tail -c 3000 gpurun_out/j13_bench_n2_gloo.log; tail -c 1500 gpurun_out/j13_bench_n1_torchrun.log; tail -c 800 gpurun_out/j13_reference.log
