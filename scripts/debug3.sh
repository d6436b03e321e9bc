cd $GRAFT_REPO_ROOT
for nw in 16 8 12 4; do for k in scalar group mat; do HQ_DEBUG_NOLANE=1 HQ_DEBUG_NW=$nw timeout 30 python scripts/debug_nw.py 60000 777 20000 $k 2>&1 | tail -1; done; done
for nw in 16 8; do for k in scalar group; do HQ_DEBUG_NOLANE=1 HQ_DEBUG_NW=$nw timeout 30 python scripts/debug_nw.py 3000000 777 2900000 $k 2>&1 | tail -1; done; done
HQ_DEBUG_NOLANE=1 HQ_DEBUG_NW=8 timeout 120 compute-sanitizer --tool synccheck python scripts/debug_nw.py 60000 777 20000 scalar 2>&1 | tail -8
