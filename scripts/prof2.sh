cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/jitsrc
export HQ_JIT_DUMP=$GRAFT_REPO_ROOT/gpurun_out/jitsrc
timeout 300 python scripts/ablate_q31.py 10
timeout 600 ncu --set full --clock-control none --import-source on -k regex:hq_jit -s 1 -c 1 -o gpurun_out/q41_sf10_v2 python scripts/profile_query.py --query ssb_q41 --sf 10 --reps 2 > gpurun_out/ncu_q41v2.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:hq_jit -s 1 -c 1 -o gpurun_out/q31_sf10_v2 python scripts/profile_query.py --query ssb_q31 --sf 10 --reps 2 > gpurun_out/ncu_q31v2.log 2>&1
ls gpurun_out/jitsrc
