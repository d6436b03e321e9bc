cd $GRAFT_REPO_ROOT
for q in "ssb_q31 30" "ssb_q41 100" "ssb_q11 30" "tpch_q6 30"; do
  set -- $q
  timeout 300 python scripts/ab_kernel.py $1 $2 11 2>&1 | tail -1
  HQ_JIT_R=4 timeout 300 python scripts/ab_kernel.py $1 $2 11 2>&1 | tail -1
  HQ_JIT_R=4 HQ_JIT_COMPACT=0 timeout 300 python scripts/ab_kernel.py $1 $2 11 2>&1 | tail -1
  HQ_JIT_R=4 HQ_JIT_NW=15 timeout 300 python scripts/ab_kernel.py $1 $2 11 2>&1 | tail -1
  HQ_JIT_NW=23 timeout 300 python scripts/ab_kernel.py $1 $2 11 2>&1 | tail -1
done
