mkdir -p gpurun_out
python -m paper_conf_ipps_00020c20_b200.build -DHGEMM_ENABLE_MC --out=/tmp/libhgemm_mc.so > /dev/null 2>&1
timeout 300 python tools/mid_variants.py base > gpurun_out/j9_mid.log 2>&1
HGEMM_EXP=32 timeout 300 python tools/mid_variants.py snake >> gpurun_out/j9_mid.log 2>&1
HGEMM_LIB=/tmp/libhgemm_mc.so HGEMM_MC=2 timeout 300 python tools/mid_variants.py mc2 >> gpurun_out/j9_mid.log 2>&1
HGEMM_LIB=/tmp/libhgemm_mc.so HGEMM_MC=1 timeout 300 python tools/mid_variants.py mcbuild_mc1 >> gpurun_out/j9_mid.log 2>&1
cat gpurun_out/j9_mid.log
