# ncu --set full of the fused kernels of TPC-H Q3 and SSB Q3.1 at SF30 (+ dumped sources)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/jitsrc
for q in tpch_q3 ssb_q31; do
  mkdir -p gpurun_out/jitsrc/$q
  HQ_JIT_DUMP=$GRAFT_REPO_ROOT/gpurun_out/jitsrc/$q timeout 600 ncu --set full --clock-control none --import-source on -k regex:hq_jit -c 4 -o gpurun_out/${q}_sf30 python scripts/profile_query.py --query $q --sf 30 --reps 1 > gpurun_out/ncu_${q}_sf30.log 2>&1
  tail -2 gpurun_out/ncu_${q}_sf30.log
  HQ_JIT_PROF=1 timeout 300 python scripts/profile_query.py --query $q --sf 30 --reps 2 2>&1 | tail -12
done
