# quick check: selected GPU tests ($1 = pytest -k expression), step timelines of TPC-H Q3 SF30 / SSB Q4.1 SF100, bench line
cd $GRAFT_REPO_ROOT
O=gpurun_out/chk; mkdir -p $O
timeout 900 python -m pytest tests -m gpu -q -x -k "${1:-queue}" > $O/tests.log 2>&1; tail -2 $O/tests.log
for qs in "tpch_q3 30" "ssb_q41 100"; do set -- $qs; timeout 600 python scripts/step_trace.py --query $1 --sf $2 > $O/trace_$1.log 2>&1; head -3 $O/trace_$1.log; grep -E 'build|rank|topk|hq_jit' $O/trace_$1.log | head -20; done
timeout 1500 python bench.py > $O/bench.json 2> $O/bench.err; python - <<'P'
import json
d=json.loads(open('gpurun_out/chk/bench.json').read().strip().splitlines()[-1])
print('value',d['value'],'ms',d['ms_per_step'],'roof',d['roofline']['frac'],d['roofline']['kernel_ms'])
for q in d.get('per_query',[]): print(q['query'],q['sf'],q['ms_per_step'],q.get('kernel_ms'))
P
