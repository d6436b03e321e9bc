cd $GRAFT_REPO_ROOT
HQ_DEBUG_NOLANE=1 HQ_DEBUG_NW=8 timeout 300 compute-sanitizer --tool memcheck --print-limit 5 python scripts/debug_nw.py 3000000 777 2900000 scalar 2>&1 | grep -v "^=========     Host Frame" | head -60
