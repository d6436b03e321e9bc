cd $GRAFT_REPO_ROOT
for q in "tpch_q10 10" "tpch_q3 30" "tpch_q18 10" "ssb_q41 30" "ssb_q31 30" "micro_groupby 10"; do
  set -- $q
  timeout 300 python scripts/ab_kernel.py $1 $2 9 2>&1 | tail -1
  HQ_JIT_ONEPASS=0 timeout 300 python scripts/ab_kernel.py $1 $2 9 2>&1 | tail -1
done
