cd $GRAFT_REPO_ROOT
timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/gpu_all.log 2>&1; tail -3 gpurun_out/gpu_all.log
timeout 600 python scripts/step_phases.py ssb_q41 100 8 2>&1 | tail -4
timeout 300 python scripts/stress_resident.py ssb_q41 30 200 2>&1 | tail -2
