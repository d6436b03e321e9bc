# ncu --set full of the small finalize kernel (SSB Q4.1 SF10, SSB Q1.1 SF10)
cd $GRAFT_REPO_ROOT
O=gpurun_out/fin; mkdir -p $O
for q in ssb_q41; do
timeout 600 ncu --set full --sampling-interval 0 --clock-control none --import-source on -k regex:finalize_small -s 2 -c 1 -o $O/$q \
  python scripts/profile_query.py --query $q --sf 10 --reps 3 > $O/$q.log 2>&1
done
ls $O
