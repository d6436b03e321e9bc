# Round 2 evidence on one B200 (run through gpurun from the repo root):
#   /usr/local/graft/bin/gpurun --timeout 5400 -- bash scripts/round02_evidence.sh
# Writes gpurun_out/r02ev/; the judged files are copied to profiles/r02/ afterwards.
cd $GRAFT_REPO_ROOT
O=gpurun_out/r02ev
mkdir -p $O
nvidia-smi --query-gpu=name,driver_version,clocks.sm,clocks.max.sm,clocks.mem --format=csv > $O/gpu.txt
timeout 1800 python -m pytest tests -m gpu -q > $O/gpu_tests.log 2>&1; tail -3 $O/gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; tail -1 $O/smoke.log
timeout 1500 python bench.py > $O/bench.json 2> $O/bench.err; tail -c 300 $O/bench.err; cut -c1-300 $O/bench.json
# launch list of the bench query (share of each kernel; cold, serialised)
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_q41.csv \
  python scripts/profile_query.py --query ssb_q41 --sf 100 --reps 2 > $O/launches_q41.log 2>&1
# ncu --set full of every bench config's fused kernel
for qs in "ssb_q41 100" "tpch_q6 10" "tpch_q1 10" "ssb_q11 10" "ssb_q12 10" "ssb_q13 10" "ssb_q31 30" "tpch_q3 30"; do
  set -- $qs
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:hq_jit -s 1 -c 1 -o $O/${1}_sf${2}_jit \
    python scripts/profile_query.py --query $1 --sf $2 --reps 2 > $O/ncu_$1.log 2>&1
done
# step timelines
for qs in "ssb_q41 100" "ssb_q11 10" "ssb_q31 30" "tpch_q3 30"; do
  set -- $qs
  timeout 600 python scripts/step_trace.py --query $1 --sf $2 --json $O/trace_$1.json > $O/trace_$1.log 2>&1
done
timeout 1200 python scripts/dist_emulate.py --query ssb_q41 --sf 100 --out $O/dist_emulate_q41.json > $O/dist_emulate.log 2>&1
timeout 1200 python scripts/micro_sweeps.py --sf 10 --reps 5 > $O/micro.log 2>&1; cp gpurun_out/micro_sweeps.* $O/ 2>/dev/null
ls $O
