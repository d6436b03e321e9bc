# Dump the NVRTC sources of every query's fused pipelines (SF1) and time them at SF10.
cd $GRAFT_REPO_ROOT
rm -rf gpurun_out/jitsrc; mkdir -p gpurun_out/jitsrc
for q in ssb_q11 ssb_q31 ssb_q41 tpch_q6 tpch_q1 tpch_q3; do
  mkdir -p gpurun_out/jitsrc/$q
  HQ_JIT_DUMP=$GRAFT_REPO_ROOT/gpurun_out/jitsrc/$q timeout 300 python scripts/profile_query.py --query $q --sf 1 --reps 1
  timeout 300 python scripts/profile_query.py --query $q --sf 10 --reps 5
done
