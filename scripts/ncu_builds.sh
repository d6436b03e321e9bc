# ncu --set full of the dimension-build kernels of SSB Q4.1 SF100 and TPC-H Q3 SF30 (one step each)
cd $GRAFT_REPO_ROOT
O=gpurun_out/nb; mkdir -p $O
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"hq_build" -s 8 -c 4 -o $O/q41_builds \
  python scripts/profile_query.py --query ssb_q41 --sf 100 --reps 3 > $O/q41.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"hq_build" -s 6 -c 3 -o $O/q3_builds \
  python scripts/profile_query.py --query tpch_q3 --sf 30 --reps 3 > $O/q3.log 2>&1
ls $O
