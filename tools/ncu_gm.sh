for g in 1 2 4 8 16; do
  timeout 300 ncu --metrics lts__t_sectors_srcunit_tex_op_read.sum,lts__t_requests_srcunit_tex_op_read.sum,lts__t_sectors_srcunit_ltcfabric.sum,dram__bytes_read.sum,gpu__time_duration.sum,gpc__cycles_elapsed.max,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed --clock-control none -k regex:hgemm_tc -s 3 -c 1 --csv python bench.py --steps 2 --warmup 3 --no-cpu --no-e2e --no-cublas --group-m $g 2>/dev/null | grep -E '^"[0-9]' | awk -v g=$g -F'","' '{print "g="g, $(NF-2), $NF}'
done
