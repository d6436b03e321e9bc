# Round evidence after the race fix: GPU tests, bench line, Q4.1 launch list and
# ncu --set full of every bench config's fused kernel, TPC-H per-query times,
# batch-processing sweep and a streamed stress run.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,driver_version,clocks.sm,clocks.max.sm,clocks.mem --format=csv > gpurun_out/gpu.txt
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/gpu_all.log 2>&1; tail -3 gpurun_out/gpu_all.log
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; tail -c 300 gpurun_out/bench.err; cut -c1-400 gpurun_out/bench.json
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_q41.csv python scripts/profile_query.py --query ssb_q41 --sf 100 --reps 2 > gpurun_out/launches_q41.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:hq_jit -s 1 -c 1 -o gpurun_out/q41_sf100_jit python scripts/profile_query.py --query ssb_q41 --sf 100 --reps 2 > gpurun_out/ncu_q41_sf100.log 2>&1
for qs in "tpch_q6 10" "tpch_q1 10" "ssb_q11 10" "ssb_q12 10" "ssb_q13 10" "ssb_q31 30" "tpch_q3 30"; do
  set -- $qs
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:hq_jit -s 1 -c 1 -o gpurun_out/${1}_sf${2}_jit python scripts/profile_query.py --query $1 --sf $2 --reps 2 > gpurun_out/ncu_$1.log 2>&1
done
timeout 900 python scripts/tpch_all.py --sf 10 > gpurun_out/tpch_all.log 2>&1; tail -3 gpurun_out/tpch_all.log
timeout 900 python scripts/stream_sweep.py --query ssb_q41 --sf 30 > gpurun_out/stream_sweep.log 2>&1; tail -3 gpurun_out/stream_sweep.log
timeout 600 python scripts/stress_stream.py ssb_q41 30 4194304 60 200 2>&1 | tail -3
timeout 900 python scripts/ssb_all.py --sf 30 --reps 5 > gpurun_out/ssb_all.log 2>&1; tail -3 gpurun_out/ssb_all.log
timeout 1800 python scripts/bytes_ratio.py --sf 10 > gpurun_out/bytes_ratio.log 2>&1; tail -3 gpurun_out/bytes_ratio.log
ls gpurun_out
