cd $GRAFT_REPO_ROOT
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -4
for qs in "tpch_q3 30" "ssb_q21 30" "ssb_q32 30" "ssb_q42 30" "ssb_q43 30" "ssb_q31 30"; do
  set -- $qs
  timeout 300 python scripts/profile_query.py --query $1 --sf $2 --reps 4 2>&1 | tail -1
done
