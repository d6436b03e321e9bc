# A/B of generator knobs (HQ_JIT_* environment variables) on the bench configs' fused kernels:
#   /usr/local/graft/bin/gpurun --timeout 1800 -- bash scripts/ab_env.sh "<query sf>;..." "<ENV=..>|<ENV=..>|..."
cd $GRAFT_REPO_ROOT
O=gpurun_out/ab; mkdir -p $O
IFS=';' read -ra QS <<< "${1:-ssb_q41 100;ssb_q41 30;ssb_q31 30}"
IFS='|' read -ra ES <<< "${2:-X=0|HQ_JIT_R=1|HQ_JIT_NW=15|HQ_JIT_NW=23}"
for qs in "${QS[@]}"; do
  for e in "${ES[@]}"; do
    r=$(env $e timeout 600 python scripts/profile_query.py --query ${qs% *} --sf ${qs#* } --reps 7 2>&1 | tail -1)
    echo "$qs | $e | $r" | tee -a $O/ab.log
  done
done
