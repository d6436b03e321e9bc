# shared-table replicas behind probes: all SSB queries at SF30 (compare with profiles/r02/ssb_all_sf30.md), Q4.1 SF100, parity subset
cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -m gpu -q -x -k "parity or golden or ssb" > /tmp/t.log 2>&1; tail -2 /tmp/t.log
python scripts/profile_query.py --query ssb_q41 --sf 100 --reps 7 2>&1 | tail -1 | sed 's/qualifying.*fused/ fused/'
timeout 1500 python scripts/ssb_all.py --sf 30 > /tmp/s.log 2>&1; cat gpurun_out/ssb_all_sf30.md | tail -14
