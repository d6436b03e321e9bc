cd $GRAFT_REPO_ROOT
timeout 120 python scripts/debug_lane.py 0.01
timeout 120 python scripts/debug_lane.py 0.01 777 20000
timeout 300 compute-sanitizer --tool memcheck python scripts/debug_lane.py 0.01 777 20000 2>&1 | tail -30
timeout 300 compute-sanitizer --tool racecheck python scripts/debug_lane.py 0.01 777 20000 2>&1 | tail -30
timeout 60 python scripts/debug_lane.py 0.1
timeout 60 python scripts/debug_lane.py 1
