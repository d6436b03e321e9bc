cd $GRAFT_REPO_ROOT
CUDA_LAUNCH_BLOCKING=1 timeout 900 python scripts/ssb_all.py --sf 30 --reps 1 --queries ssb_q13,ssb_q21 2>&1 | grep -v "^    " | tail -8
CUDA_LAUNCH_BLOCKING=1 timeout 900 python scripts/ssb_all.py --sf 30 --reps 1 --queries ssb_q21 2>&1 | grep -v "^    " | tail -4
