cd $GRAFT_REPO_ROOT
HQ_MP_DEBUG=1 timeout 900 python scripts/ssb_all.py --sf 30 --reps 1 --queries ssb_q13,ssb_q21 2>&1 | grep -v "^    " | grep -v "^  File" | tail -12
HQ_MP_DEBUG=1 timeout 900 python scripts/ssb_all.py --sf 30 --reps 1 --queries ssb_q21 2>&1 | grep "hq multipass" | tail -3
