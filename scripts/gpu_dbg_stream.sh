cd $GRAFT_REPO_ROOT
timeout 600 python scripts/dbg_stream.py ssb_q41 30 1048576,4194304,8388608 2>&1 | tail -20
timeout 300 python scripts/dbg_stream.py tpch_q6 10 4194304,16777216 2>&1 | tail -8
timeout 300 python scripts/dbg_stream.py ssb_q41 10 4194304 nopin 2>&1 | tail -6
