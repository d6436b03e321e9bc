# A/B: early stage release (HQ_JIT_EARLY) x rows per lane, kernel times per query
cd $GRAFT_REPO_ROOT
for cfg in "0 2" "1 2" "1 4" "0 4"; do
  set -- $cfg; E=$1; RR=$2
  echo "== EARLY=$E R=$RR"
  for qs in "tpch_q3 30" "ssb_q31 30" "ssb_q41 100" "tpch_q6 10" "ssb_q11 10" "tpch_q1 10"; do
    set -- $qs
    HQ_JIT_EARLY=$E HQ_JIT_R=$RR timeout 300 python scripts/profile_query.py --query $1 --sf $2 --reps 4 2>&1 | tail -1
  done
done
