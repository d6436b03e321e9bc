cd $GRAFT_REPO_ROOT
for q in "tpch_q10 10" "ssb_q41 100" "ssb_q31 30" "tpch_q3 30"; do
  set -- $q
  timeout 300 python scripts/ab_kernel.py $1 $2 9 2>&1 | tail -1
done
timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/gpu_all.log 2>&1; tail -2 gpurun_out/gpu_all.log
timeout 600 python scripts/tpch_all.py --sf 10 --queries tpch_q18,tpch_q21,tpch_q10 > gpurun_out/t.log 2>&1; tail -5 gpurun_out/t.log
