# GPU tests, the bench line, the launch list and ncu captures for profiles/
cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
bash scripts/bench_and_profile.sh
timeout 900 python scripts/bytes_ratio.py > gpurun_out/bytes_ratio.log 2>&1; tail -3 gpurun_out/bytes_ratio.log
