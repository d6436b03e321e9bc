cd $GRAFT_REPO_ROOT
timeout 600 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
for w in suspend sleep; do
  echo "== WAIT=$w"
  for qs in "ssb_q31 30" "ssb_q41 100" "tpch_q3 30" "ssb_q11 10" "tpch_q6 10" "tpch_q1 10"; do
    set -- $qs
    HQ_JIT_WAIT=$w timeout 300 python scripts/profile_query.py --query $1 --sf $2 --reps 4 2>&1 | tail -1
  done
done
for nwr in "16 4" "24 4" "31 1"; do set -- $nwr; echo "== NW=$1 R=$2 nocompact"; for q in ssb_q31 ssb_q41; do HQ_JIT_COMPACT=0 HQ_JIT_NW=$1 HQ_JIT_R=$2 timeout 300 python scripts/profile_query.py --query $q --sf 30 --reps 4 2>&1 | tail -1; done; done
