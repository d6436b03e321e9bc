cd $GRAFT_REPO_ROOT
timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/gpu_all.log 2>&1; tail -3 gpurun_out/gpu_all.log
timeout 900 python scripts/tpch_all.py --sf 10 > gpurun_out/tpch_all.log 2>&1; tail -14 gpurun_out/tpch_all.log
timeout 300 python scripts/stress_resident.py ssb_q41 30 300 2>&1 | tail -2
timeout 600 python scripts/ssb_all.py --sf 30 --reps 3 > gpurun_out/ssb_all.log 2>&1; tail -16 gpurun_out/ssb_all.log
