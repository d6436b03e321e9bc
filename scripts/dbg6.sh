cd $GRAFT_REPO_ROOT
git -C $GRAFT_REPO_ROOT stash list >/dev/null 2>&1
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
timeout 1500 python scripts/ssb_all.py --sf 30 --reps 5 2>&1 | tail -16
