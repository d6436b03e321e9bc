cd $GRAFT_REPO_ROOT
timeout 300 python scripts/ablate_q41.py 10
timeout 120 python scripts/profile_query.py --query ssb_q31 --sf 10 --reps 3 2>&1 | tail -1
