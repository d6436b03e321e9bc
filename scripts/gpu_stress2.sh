cd $GRAFT_REPO_ROOT
HQ_JIT_RELFIX=none timeout 600 python scripts/stress_resident.py ssb_q41 30 500 2>&1 | tail -4
HQ_JIT_RELFIX=fence timeout 600 python scripts/stress_resident.py ssb_q41 30 500 2>&1 | tail -4
timeout 900 python scripts/stress_resident.py ssb_q41 30 1000 2>&1 | tail -4
