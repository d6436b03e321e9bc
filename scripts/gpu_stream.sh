# Streaming parity + whole GPU suite + TPC-H per-query times + streaming sweep
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_stream.py -x -q > gpurun_out/gpu_stream.log 2>&1; tail -25 gpurun_out/gpu_stream.log
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/gpu_all.log 2>&1; tail -5 gpurun_out/gpu_all.log
timeout 900 python scripts/tpch_all.py --sf 10 > gpurun_out/tpch_all.log 2>&1; tail -16 gpurun_out/tpch_all.log
timeout 900 python scripts/stream_sweep.py --query ssb_q41 --sf 30 > gpurun_out/stream_sweep.log 2>&1; tail -12 gpurun_out/stream_sweep.log
