cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "q9 or f3" > gpurun_out/gpu_q9.log 2>&1; tail -25 gpurun_out/gpu_q9.log
timeout 900 python -m pytest tests/test_gpu_dist.py -x -q > gpurun_out/gpu_dist.log 2>&1; tail -8 gpurun_out/gpu_dist.log
timeout 600 python scripts/tpch_all.py --sf 10 --queries tpch_q9,tpch_q10 > gpurun_out/tpch_q9.log 2>&1; tail -5 gpurun_out/tpch_q9.log
