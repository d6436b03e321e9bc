cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,driver_version,clocks.sm,clocks.max.sm,clocks.mem --format=csv > gpurun_out/gpu.txt
timeout 900 python bench.py > gpurun_out/bench_r01.json 2> gpurun_out/bench_r01.err
tail -c 3000 gpurun_out/bench_r01.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_q41.csv python scripts/profile_query.py --query ssb_q41 --sf 100 --reps 2 > gpurun_out/launches_q41.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:hq_jit -s 1 -c 1 -o gpurun_out/q41_sf100_jit python scripts/profile_query.py --query ssb_q41 --sf 100 --reps 2 > gpurun_out/ncu_q41_sf100.log 2>&1
for q in tpch_q6 tpch_q1 ssb_q11 ssb_q31 tpch_q3; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:hq_jit -s 1 -c 1 -o gpurun_out/${q}_jit python scripts/profile_query.py --query $q --sf 10 --reps 2 > gpurun_out/ncu_$q.log 2>&1
done
ls gpurun_out
