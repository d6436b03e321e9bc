cd $GRAFT_REPO_ROOT
O=gpurun_out/r02ev
mkdir -p $O
for x in 32 512 2048 8192; do timeout 300 python scripts/profile_query.py --query micro_groupby --sf 10 --reps 3 --kw x=$x 2>&1 | tail -1; done
timeout 1200 python scripts/micro_sweeps.py --sf 10 --reps 5 > $O/micro.log 2>&1; cp gpurun_out/micro_sweeps.* $O/ 2>/dev/null; tail -12 $O/micro_sweeps.md
timeout 3600 python scripts/bytes_ratio.py --queries ssb_q41:100,ssb_q31:30,tpch_q3:30,tpch_q1:10,tpch_q6:10,ssb_q11:10 \
  > $O/bytes_ratio.log 2>&1; cp gpurun_out/bytes_ratio_bench_sfs.* $O/ 2>/dev/null
# compute-sanitizer on the SF 0.01 configs (memcheck, racecheck, synccheck)
for tool in memcheck racecheck synccheck; do
  for q in ssb_q41 ssb_q31 tpch_q3 tpch_q6; do
    timeout 900 compute-sanitizer --tool $tool --print-limit 20 python scripts/profile_query.py --query $q --sf 0.01 --reps 1 \
      > $O/sanitizer_${tool}_${q}.log 2>&1
    tail -2 $O/sanitizer_${tool}_${q}.log
  done
done
ls $O
# the distributed code path at world size 1 (NCCL, torchrun): its fixed cost over the single-device engine
HQ_FORCE_DIST=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 \
  --master-port 29561 bench.py --no-extra --steps 10 --warmup 3 > $O/bench_forcedist.json 2> $O/bench_forcedist.err
HQ_BENCH_EAGER=1 timeout 900 python bench.py --no-extra --steps 10 --warmup 3 > $O/bench_eager.json 2> $O/bench_eager.err
cut -c1-300 $O/bench_forcedist.json $O/bench_eager.json
