cd $GRAFT_REPO_ROOT
timeout 600 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
for qs in "ssb_q31 30" "ssb_q41 100" "tpch_q3 30" "ssb_q11 10" "tpch_q6 10" "tpch_q1 10"; do
  set -- $qs
  timeout 300 python scripts/profile_query.py --query $1 --sf $2 --reps 4 2>&1 | tail -1
done
for q in tpch_q1 ssb_q41 ssb_q31; do timeout 300 python scripts/profile_query.py --query $q --sf 10 --reps 2 --exec oaat 2>&1 | tail -1; done
