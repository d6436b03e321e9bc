cd $GRAFT_REPO_ROOT
timeout 900 compute-sanitizer --tool memcheck --print-limit 3 python scripts/ssb_all.py --sf 1 --reps 1 --queries ssb_q13,ssb_q21 2>&1 | grep -v "^=========     " | head -40
