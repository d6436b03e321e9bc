cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
for qs in "ssb_q31 30" "ssb_q41 100" "tpch_q1 10" "ssb_q11 10"; do
  set -- $qs
  timeout 300 python scripts/profile_query.py --query $1 --sf $2 --reps 4 2>&1 | tail -1
done
timeout 1200 python scripts/micro_sweeps.py --sf 10 --reps 7 2>&1 | tail -22
