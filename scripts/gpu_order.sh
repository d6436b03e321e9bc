cd $GRAFT_REPO_ROOT
for o in scd sdc dsc csd; do timeout 300 python scripts/ab_kernel.py ssb_q31 30 9 porder=$o 2>&1 | tail -1; done
