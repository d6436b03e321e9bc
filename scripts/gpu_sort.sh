cd $GRAFT_REPO_ROOT
timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/gpu_all.log 2>&1; tail -2 gpurun_out/gpu_all.log
timeout 300 python scripts/step_phases.py tpch_q3 30 6 2>&1 | tail -3
timeout 600 python scripts/tpch_all.py --sf 10 --queries tpch_q3,tpch_q10,tpch_q18 > gpurun_out/t.log 2>&1; tail -4 gpurun_out/t.log
