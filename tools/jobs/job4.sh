# launch/teardown probes, sustained-regime comparison vs cuBLAS (incl. multicast build)
mkdir -p gpurun_out
O=gpurun_out/j4
timeout 300 python tools/teardown_probe.py > $O.teardown.log 2>&1
for e in 4 8 16 28; do HGEMM_EXP=$e timeout 120 python tools/teardown_probe.py --gemm-only >> $O.teardown.log 2>&1; done
HGEMM_PDL=0 timeout 120 python tools/teardown_probe.py --gemm-only >> $O.teardown.log 2>&1
timeout 300 python tools/sustained.py --m 16384 --warm 3 --iters 150 > $O.sustained.log 2>&1
timeout 300 python tools/sustained.py --m 16384 --warm 3 --iters 150 --compute f16 --order ours >> $O.sustained.log 2>&1
timeout 300 python tools/sustained.py --m 32768 --warm 3 --iters 20 --order ours,cublas >> $O.sustained.log 2>&1
python -m paper_conf_ipps_00020c20_b200.build -DHGEMM_ENABLE_MC --out=/tmp/libhgemm_mc.so > /dev/null 2>&1
HGEMM_LIB=/tmp/libhgemm_mc.so HGEMM_MC=2 timeout 300 python tools/sustained.py --m 16384 --warm 3 --iters 150 --order ours >> $O.sustained.log 2>&1
tail -n 40 $O.*.log
