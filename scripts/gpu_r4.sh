cd $GRAFT_REPO_ROOT
for q in "ssb_q11 30" "ssb_q12 30" "ssb_q13 30" "ssb_q31 30" "ssb_q41 100" "tpch_q6 30" "tpch_q1 30" "ssb_q21 30" "micro_sum 30"; do
  set -- $q
  timeout 300 python scripts/ab_kernel.py $1 $2 11 2>&1 | tail -1
done
timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/gpu_all.log 2>&1; tail -3 gpurun_out/gpu_all.log
