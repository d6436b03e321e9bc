# GPU tests, then per-query SF10 kernel times and dumped sources (SF1)
cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -15
bash scripts/dump_src.sh 2>&1 | grep -v "^loaded" | grep " 10.0 "
