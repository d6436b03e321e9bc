cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -4
for qs in "ssb_q31 10" "ssb_q41 10" "tpch_q3 10" "ssb_q11 10" "tpch_q6 10" "tpch_q1 10" "ssb_q31_mat 10"; do
  set -- $qs
  for e in fused multipass oaat; do timeout 300 python scripts/profile_query.py --query $1 --sf $2 --reps 3 --exec $e 2>&1 | tail -1 | sed "s/^/$e /"; done
done
