cd $GRAFT_REPO_ROOT
timeout 1500 compute-sanitizer --tool memcheck --print-limit 4 python scripts/ssb_all.py --sf 30 --reps 1 --queries ssb_q13,ssb_q21 2>&1 | grep -v "^    " | head -60
