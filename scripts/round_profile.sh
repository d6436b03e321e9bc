# Round evidence on one B200: GPU tests, the bench line, the launch list of the
# bench command's query, ncu --set full of every bench config's fused kernel,
# the fused / multi-pass / op-at-a-time DRAM-bytes table and the micro sweeps.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,driver_version,clocks.sm,clocks.max.sm,clocks.mem --format=csv > gpurun_out/gpu.txt
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
timeout 1200 python bench.py > gpurun_out/bench_r01.json 2> gpurun_out/bench_r01.err; tail -c 600 gpurun_out/bench_r01.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_q41.csv python scripts/profile_query.py --query ssb_q41 --sf 100 --reps 2 > gpurun_out/launches_q41.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:hq_jit -s 1 -c 1 -o gpurun_out/q41_sf100_jit python scripts/profile_query.py --query ssb_q41 --sf 100 --reps 2 > gpurun_out/ncu_q41_sf100.log 2>&1
for qs in "tpch_q6 10" "tpch_q1 10" "ssb_q11 10" "ssb_q12 10" "ssb_q13 10" "ssb_q31 30" "tpch_q3 30"; do
  set -- $qs
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:hq_jit -s 1 -c 1 -o gpurun_out/${1}_sf${2}_jit python scripts/profile_query.py --query $1 --sf $2 --reps 2 > gpurun_out/ncu_$1.log 2>&1
done
timeout 2400 python scripts/bytes_ratio.py --sf 10 > gpurun_out/bytes_ratio.log 2>&1; tail -14 gpurun_out/bytes_ratio.log
timeout 900 python scripts/micro_sweeps.py --sf 10 --reps 7 > gpurun_out/micro.log 2>&1; tail -3 gpurun_out/micro.log
ls gpurun_out
