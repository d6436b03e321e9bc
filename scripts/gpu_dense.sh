cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "f3 or q9 or q21" > gpurun_out/p.log 2>&1; tail -3 gpurun_out/p.log
timeout 900 python -m pytest tests/test_gpu_dist.py -q -x 2>&1 | tail -3
timeout 900 python scripts/tpch_all.py --sf 10 > gpurun_out/tpch_all.log 2>&1; tail -16 gpurun_out/tpch_all.log
