cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/jitsrc
timeout 900 python bench.py > gpurun_out/bench_r01b.json 2> gpurun_out/bench_r01b.err
tail -c 1500 gpurun_out/bench_r01b.err
HQ_JIT_DUMP=$GRAFT_REPO_ROOT/gpurun_out/jitsrc timeout 900 ncu --set full --clock-control none --import-source on -k regex:hq_jit -s 1 -c 1 -o gpurun_out/q41_sf100_v3 python scripts/profile_query.py --query ssb_q41 --sf 100 --reps 2 > gpurun_out/ncu_q41v3.log 2>&1
HQ_JIT_DUMP=$GRAFT_REPO_ROOT/gpurun_out/jitsrc timeout 900 ncu --set full --clock-control none --import-source on -k regex:hq_jit -s 1 -c 1 -o gpurun_out/q31_sf30_v3 python scripts/profile_query.py --query ssb_q31 --sf 30 --reps 2 > gpurun_out/ncu_q31v3.log 2>&1
