cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -4
HQ_FORCE_DIST=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29534 bench.py --gpus 1 --steps 3 --warmup 3 --sf 1 --no-extra 2>&1 | tail -3 | cut -c1-600
for q in ssb_q31 ssb_q41 tpch_q3; do timeout 120 python scripts/profile_query.py --query $q --sf 10 --reps 3 2>&1 | tail -1; done
