cd $GRAFT_REPO_ROOT
timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/gpu_all.log 2>&1; tail -3 gpurun_out/gpu_all.log
timeout 900 python scripts/tpch_all.py --sf 10 > gpurun_out/tpch_all.log 2>&1; tail -16 gpurun_out/tpch_all.log
