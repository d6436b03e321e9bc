# TPC-H Q3 SF30: generated kernels (HQ_JIT_DUMP) + ncu --set full of the build / top-k kernels of one step
cd $GRAFT_REPO_ROOT
O=gpurun_out/q3; mkdir -p $O/src
HQ_JIT_DUMP=$O/src timeout 600 python scripts/profile_query.py --query tpch_q3 --sf 30 --reps 3 > $O/run.log 2>&1; tail -1 $O/run.log
timeout 900 ncu --set full --clock-control none -k regex:"hq_build|hq_rank|hq_topk|hq_init" -s 30 -c 16 -o $O/q3_aux \
  python scripts/profile_query.py --query tpch_q3 --sf 30 --reps 3 > $O/ncu_aux.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:hq_jit -s 4 -c 2 -o $O/q3_jit \
  python scripts/profile_query.py --query tpch_q3 --sf 30 --reps 3 > $O/ncu_jit.log 2>&1
ls $O
