cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/jitsrc/q31b
HQ_JIT_DUMP=$GRAFT_REPO_ROOT/gpurun_out/jitsrc/q31b timeout 600 ncu --set full --clock-control none --import-source on -k regex:hq_jit -c 1 -o gpurun_out/q31b python scripts/profile_query.py --query ssb_q31 --sf 30 --reps 1 > gpurun_out/ncu_q31b.log 2>&1
tail -1 gpurun_out/ncu_q31b.log
mkdir -p gpurun_out/jitsrc/q41b
HQ_JIT_DUMP=$GRAFT_REPO_ROOT/gpurun_out/jitsrc/q41b timeout 600 ncu --set full --clock-control none --import-source on -k regex:hq_jit -c 1 -o gpurun_out/q41b python scripts/profile_query.py --query ssb_q41 --sf 100 --reps 1 > gpurun_out/ncu_q41b.log 2>&1
tail -1 gpurun_out/ncu_q41b.log
