set -x
cd $GRAFT_REPO_ROOT
python scripts/profile_query.py --query ssb_q41 --sf 10 --reps 3
python scripts/profile_query.py --query tpch_q1 --sf 10 --reps 3
timeout 600 ncu --set full --clock-control none --import-source on -k regex:hq_fused -s 1 -c 1 -o gpurun_out/q41_full python scripts/profile_query.py --query ssb_q41 --sf 10 --reps 2 > gpurun_out/ncu_q41.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:hq_fused -s 1 -c 1 -o gpurun_out/q1_full python scripts/profile_query.py --query tpch_q1 --sf 10 --reps 2 > gpurun_out/ncu_q1.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:hq_fused -s 1 -c 1 -o gpurun_out/q6_full python scripts/profile_query.py --query tpch_q6 --sf 10 --reps 2 > gpurun_out/ncu_q6.log 2>&1
ls -la gpurun_out
