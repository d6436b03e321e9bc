import sys, os, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import hqgen, oracle
from paper_conf_sigmod_funkebnmt18_b200 import hq
from paper_conf_sigmod_funkebnmt18_b200.engine import Engine
from paper_conf_sigmod_funkebnmt18_b200.queries import QUERIES, load_tables
sf = float(sys.argv[1]); fr = None
if len(sys.argv) > 3: fr = (int(sys.argv[2]), int(sys.argv[3]))
ctx = hq.Context(0)
host = {t: hqgen.generate(t, sf) for t in hqgen.TPCH_TABLES}
q = QUERIES["tpch_q1"]
E = Engine(ctx, load_tables(ctx, q, sf, host=host), fact_range=fr)
t0 = time.time()
g = q.execute(E)
print("gpu", time.time() - t0, g.rows(["l_returnflag", "l_linestatus", "count_order"]), flush=True)
li = host["lineitem"]
if fr: li = {k: v[fr[0]:fr[1]] for k, v in li.items()}
o = oracle.tpch_q1(li)
print("orc", o.rows(["l_returnflag", "l_linestatus", "count_order"]))
