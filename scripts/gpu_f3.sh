# GPU parity of the f3 TPC-H queries, then the whole GPU suite
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "f3 or q21_appf or q7" > gpurun_out/gpu_f3.log 2>&1; tail -30 gpurun_out/gpu_f3.log
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/gpu_all.log 2>&1; tail -5 gpurun_out/gpu_all.log
