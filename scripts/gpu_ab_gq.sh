# warp update queues (HQ_JIT_NOGQ=1: off): TPC-H Q3 lineitem pipeline and the GROUP BY orderkey queries
cd $GRAFT_REPO_ROOT
for e in X=0 HQ_JIT_NOGQ=1; do echo $e; env $e python scripts/ablate_tpch_q3.py 30 2>&1 | tail -1;
  for q in tpch_q3 tpch_q10 tpch_q18 tpch_q21 tpch_q13 tpch_q4; do env $e python scripts/profile_query.py --query $q --sf 10 --reps 5 2>&1 | tail -1 | sed 's/qualifying.*fused/ fused/'; done; done
timeout 1800 python -m pytest tests -m gpu -q -x > gpurun_out/gq_tests.log 2>&1; tail -3 gpurun_out/gq_tests.log
