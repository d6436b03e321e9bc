cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -4
for q in ssb_q31 ssb_q41 tpch_q3 tpch_q1 micro_groupby; do timeout 120 python scripts/profile_query.py --query $q --sf 10 --reps 3 2>&1 | tail -1; done
for r in 4; do HQ_JIT_R=$r timeout 120 python scripts/profile_query.py --query ssb_q31 --sf 10 --reps 3 2>&1 | tail -1; done
