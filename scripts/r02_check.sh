# round-2 validation call: GPU tests, the distributed engine at world size 1 vs eager,
# lazy loads of SSB Q1.2 / Q1.3 (source-row pass estimate)
cd $GRAFT_REPO_ROOT
O=gpurun_out/r02chk4
mkdir -p $O
timeout 2400 python -m pytest tests -m gpu -q -x > $O/gpu_tests.log 2>&1; tail -3 $O/gpu_tests.log
HQ_FORCE_DIST=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 \
  --master-port 29561 bench.py --no-extra --steps 10 --warmup 3 > $O/bench_forcedist.json 2> $O/bench_forcedist.err
HQ_BENCH_EAGER=1 timeout 900 python bench.py --no-extra --steps 10 --warmup 3 > $O/bench_eager.json 2> $O/bench_eager.err
cut -c1-200 $O/bench_forcedist.json $O/bench_eager.json
timeout 600 python scripts/step_trace.py --query ssb_q41 --sf 100 --dist > $O/trace_ssb_q41_dist.log 2>&1; grep -m3 '^step' $O/trace_ssb_q41_dist.log
for q in ssb_q11 ssb_q12 ssb_q13 ssb_q21 ssb_q31 tpch_q6; do
  timeout 300 python scripts/profile_query.py --query $q --sf 10 --reps 7 2>&1 | tail -1
  timeout 600 ncu --metrics dram__bytes_read.sum,gpu__time_duration.sum --clock-control none \
    -k regex:hq_jit -s 2 -c 1 --csv python scripts/profile_query.py --query $q --sf 10 --reps 3 > $O/ncu_lazy_$q.csv 2>&1
  grep -E 'dram__bytes_read.sum|gpu__time_duration.sum' $O/ncu_lazy_$q.csv | awk -F'","' '{print $(NF-2), $NF}' | tr '\n' ' '; echo
done
