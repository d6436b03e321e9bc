# TPC-H per-query measurements at SF10 on one B200
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,driver_version,clocks.sm,clocks.max.sm,clocks.mem --format=csv > gpurun_out/gpu.txt
timeout 1500 python scripts/tpch_all.py --sf 10 > gpurun_out/tpch_all.log 2>&1; tail -20 gpurun_out/tpch_all.log
