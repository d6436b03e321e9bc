cd $GRAFT_REPO_ROOT
echo "== lane default"; timeout 60 python scripts/debug_lane.py 1
echo "== nolane nw16"; HQ_DEBUG_NOLANE=1 timeout 60 python scripts/debug_lane.py 1
echo "== nolane nw8"; HQ_DEBUG_NOLANE=1 HQ_DEBUG_NW=8 timeout 60 python scripts/debug_lane.py 1
echo "== lane nw16"; HQ_DEBUG_NW=16 timeout 60 python scripts/debug_lane.py 1
echo "== nolane nw8 part"; HQ_DEBUG_NOLANE=1 HQ_DEBUG_NW=8 timeout 60 python scripts/debug_lane.py 0.01 777 20000
