# ncu --set full of the fused kernel of two star-join queries (current code)
cd $GRAFT_REPO_ROOT
TAG=${TAG:-v4}
for q in ssb_q41 ssb_q31; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:hq_jit -s 1 -c 1 -o gpurun_out/${q}_sf10_$TAG python scripts/profile_query.py --query $q --sf 10 --reps 2 > gpurun_out/ncu_${q}_$TAG.log 2>&1
  tail -2 gpurun_out/ncu_${q}_$TAG.log
done
