cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "f3 or q9 or q21" > gpurun_out/p.log 2>&1; tail -3 gpurun_out/p.log
timeout 900 python -m pytest tests/test_gpu_dist.py -q -x > gpurun_out/d.log 2>&1; tail -3 gpurun_out/d.log
timeout 600 python scripts/step_phases.py tpch_q18 10 5 2>&1 | tail -3
timeout 600 python scripts/tpch_all.py --sf 10 --queries tpch_q13,tpch_q18,tpch_q21 > gpurun_out/tpch_sub.log 2>&1; tail -6 gpurun_out/tpch_sub.log
