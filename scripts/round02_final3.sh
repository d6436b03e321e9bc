# Round 2 final measurements on one B200 (through gpurun from the repo root):
#   /usr/local/graft/bin/gpurun --timeout 5400 -- bash scripts/round02_final3.sh
# Writes gpurun_out/r02fin3/; the judged files are copied to profiles/r02/ afterwards.
cd $GRAFT_REPO_ROOT
O=gpurun_out/r02fin3
mkdir -p $O
nvidia-smi --query-gpu=name,driver_version,clocks.sm,clocks.max.sm,clocks.mem --format=csv > $O/gpu.txt
timeout 1800 python -m pytest tests -m gpu -q > $O/gpu_tests.log 2>&1; tail -3 $O/gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; tail -1 $O/smoke.log
timeout 1500 python bench.py > $O/bench.json 2> $O/bench.err; tail -c 300 $O/bench.err; cut -c1-300 $O/bench.json
timeout 900 python bench.py --impl reference --steps 3 --warmup 3 > $O/bench_ref.json 2> $O/bench_ref.err; cut -c1-200 $O/bench_ref.json
# launch list of the bench query (share of each kernel; cold, serialised)
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_q41.csv \
  python scripts/profile_query.py --query ssb_q41 --sf 100 --reps 2 > $O/launches_q41.log 2>&1
# ncu --set full of every bench config's fused kernel (TPC-H Q3: its lineitem pipeline)
for qs in "ssb_q41 100 1" "ssb_q31 30 1" "tpch_q3 30 1"; do
  set -- $qs
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:hq_jit -s $3 -c 1 -o $O/${1}_sf${2}_jit \
    python scripts/profile_query.py --query $1 --sf $2 --reps 2 > $O/ncu_$1.log 2>&1
done
for qs in "ssb_q41 100" "ssb_q31 30" "tpch_q3 30" "ssb_q11 10"; do
  set -- $qs
  timeout 600 python scripts/step_trace.py --query $1 --sf $2 --json $O/trace_$1.json > $O/trace_$1.log 2>&1
done
timeout 600 python scripts/step_trace.py --query ssb_q41 --sf 100 --dist > $O/trace_ssb_q41_dist.log 2>&1
HQ_FORCE_DIST=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 \
  --master-port 29561 bench.py --no-extra --steps 10 --warmup 3 > $O/bench_forcedist.json 2> $O/bench_forcedist.err
timeout 1200 python scripts/dist_emulate.py --query ssb_q41 --sf 100 --out $O/dist_emulate_q41.json > $O/dist_emulate.log 2>&1
timeout 1200 python scripts/dist_emulate.py --query tpch_q3 --sf 30 --out $O/dist_emulate_tpch_q3.json > $O/dist_emulate_q3.log 2>&1
timeout 1800 python scripts/ssb_all.py --sf 30 > $O/ssb_all.log 2>&1; cp gpurun_out/ssb_all_sf30.* $O/ 2>/dev/null
timeout 1800 python scripts/tpch_all.py --sf 10 > $O/tpch_all.log 2>&1; cp gpurun_out/tpch_all_sf10.* $O/ 2>/dev/null
ls $O
