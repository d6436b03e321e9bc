cd $GRAFT_REPO_ROOT
for q in "ssb_q41 100" "ssb_q31 30" "tpch_q3 30"; do
  set -- $q
  for v in dep fence none; do HQ_JIT_RELFIX=$v timeout 300 python scripts/ab_kernel.py $1 $2 15 2>&1 | tail -1; done
  HQ_JIT_EARLY=0 timeout 300 python scripts/ab_kernel.py $1 $2 15 2>&1 | tail -1
done
HQ_JIT_RELFIX=fence timeout 900 python scripts/stress_resident.py ssb_q41 30 1500 2>&1 | tail -2
timeout 900 python scripts/stress_resident.py ssb_q41 30 1500 2>&1 | tail -2
