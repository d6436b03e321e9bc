cd $GRAFT_REPO_ROOT
for cfg in "16 4" "16 2" "24 2" "24 4" "31 2" "31 1" "8 8"; do
  set -- $cfg
  echo "== NW=$1 R=$2"
  for q in ssb_q31 ssb_q41 tpch_q3 tpch_q6; do HQ_JIT_NW=$1 HQ_JIT_R=$2 timeout 120 python scripts/profile_query.py --query $q --sf 10 --reps 3 2>&1 | tail -1; done
done
