cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/lay
timeout 900 python scripts/exp_col_layout.py --query ssb_q41 --sf 100 > gpurun_out/lay/q41_sf100.log 2>&1; cat gpurun_out/lay/q41_sf100.log | head -8
timeout 600 python scripts/exp_col_layout.py --query ssb_q41 --sf 30 > gpurun_out/lay/q41_sf30.log 2>&1; cat gpurun_out/lay/q41_sf30.log | head -8
timeout 600 python scripts/exp_col_layout.py --query ssb_q31 --sf 30 > gpurun_out/lay/q31_sf30.log 2>&1; cat gpurun_out/lay/q31_sf30.log | head -8
