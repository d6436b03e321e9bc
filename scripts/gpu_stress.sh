cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/dump
HQ_JIT_DUMP=gpurun_out/dump timeout 300 python scripts/stress_resident.py ssb_q41 30 2 2>&1 | tail -2
timeout 1500 python scripts/stress_resident.py ssb_q41 30 300 "" HQ_JIT_EARLY=0 HQ_JIT_NOLOCAL=1 HQ_JIT=0 HQ_JIT_R=1 HQ_JIT_WAIT=sleep 2>&1 | tail -24
