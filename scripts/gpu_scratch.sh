cd $GRAFT_REPO_ROOT
timeout 300 python scripts/exp_rerun.py ssb_q31 10 16 2
for q in ssb_q41; do timeout 300 python scripts/exp_rerun.py $q 10 16 1; done
timeout 300 python scripts/exp_rerun.py tpch_q3 10 4 1
HQ_JIT_PROF=1 timeout 300 python scripts/exp_rerun.py ssb_q31 10 4 1 2>&1 | grep "CTAs >"
