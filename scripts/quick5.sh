cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -15
for q in tpch_q6 tpch_q1 ssb_q11 ssb_q31 ssb_q41 tpch_q3 micro_groupby; do timeout 120 python scripts/profile_query.py --query $q --sf 10 --reps 3 2>&1 | tail -1; done
