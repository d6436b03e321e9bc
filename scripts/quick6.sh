cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -15
timeout 1800 python scripts/bytes_ratio.py --sf 10 --round r01 2>&1 | tail -14
