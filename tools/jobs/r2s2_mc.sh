mkdir -p gpurun_out
export HGEMM_LIB=ab_libs/mc.so
for mcv in 1 2; do
  HGEMM_MC=$mcv python tools/lts_probe.py > /dev/null 2>&1 || echo "plain failed"
  HGEMM_MC=$mcv ncu --metrics gpu__time_duration.sum,lts__t_sectors_srcunit_tex_op_read.sum,launch__cluster_dim_x --clock-control none --csv --log-file gpurun_out/mc_probe_$mcv.csv python tools/lts_probe.py > gpurun_out/mc_probe_order_$mcv.txt 2>/dev/null
  echo "== HGEMM_MC=$mcv"; python tools/launch_cost_join.py gpurun_out/mc_probe_$mcv.csv gpurun_out/mc_probe_order_$mcv.txt
done
