cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -m gpu -q -x -k "parity or golden or edge or guard or micro or we" > /tmp/t.log 2>&1; tail -2 /tmp/t.log
for q in ssb_q41 ssb_q31 ssb_q11 tpch_q1; do python scripts/step_trace.py --query $q --sf 10 2>&1 | grep finalize | tail -1; done
