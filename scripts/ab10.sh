cd $GRAFT_REPO_ROOT
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
timeout 300 python scripts/profile_query.py --query tpch_q3 --sf 30 --reps 4 2>&1 | tail -1
timeout 1500 python scripts/ssb_all.py --sf 30 --reps 5 2>&1 | tail -17
