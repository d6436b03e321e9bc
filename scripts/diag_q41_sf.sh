# Q4.1 SF30 vs SF100: the generated kernels (HQ_JIT_DUMP) and ncu memory / stall metrics
#   /usr/local/graft/bin/gpurun --timeout 2400 -- bash scripts/diag_q41_sf.sh
cd $GRAFT_REPO_ROOT
O=gpurun_out/diag41
mkdir -p $O/src30 $O/src100
HQ_JIT_DUMP=$O/src30 timeout 600 python scripts/profile_query.py --query ssb_q41 --sf 30 --reps 7 > $O/run30.log 2>&1; tail -1 $O/run30.log
HQ_JIT_DUMP=$O/src100 timeout 600 python scripts/profile_query.py --query ssb_q41 --sf 100 --reps 7 > $O/run100.log 2>&1; tail -1 $O/run100.log
M=gpu__time_duration.sum,dram__bytes_read.sum,lts__t_sector_hit_rate.pct,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sectors_srcunit_tex_op_read_lookup_hit.sum,l1tex__t_sector_hit_rate.pct,smsp__average_warp_latency_issue_stalled_long_scoreboard.ratio,smsp__inst_executed.sum,sm__warps_active.avg.pct_of_peak_sustained_active,smsp__issue_active.avg.pct_of_peak_sustained_active,l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum,lts__average_t_sector_hit_rate_realtime.pct,lts__t_sectors_srcnode_fbp.sum
for sf in 30 100; do
  timeout 900 ncu --metrics $M --clock-control none -k regex:hq_jit -s 2 -c 1 --csv \
    python scripts/profile_query.py --query ssb_q41 --sf $sf --reps 3 > $O/ncu_$sf.csv 2> $O/ncu_$sf.err
done
ls $O
