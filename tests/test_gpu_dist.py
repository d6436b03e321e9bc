"""Multi-rank execution through the real device engine: two processes share
cuda:0 (gloo moves the CUDA buffers; NCCL refuses two ranks on one device), so
the root-build + broadcast + hq_hash_import + partial-reduce path of
dist.DistributedEngine runs end to end on the GPU.  Each rank owns a range
partition of the fact table; the root's result must equal the oracle."""
import os
import socket

import pytest
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu

SF = 0.01
QS = ["ssb_q41", "ssb_q31", "ssb_q11", "tpch_q6", "tpch_q1", "tpch_q3", "tpch_q5", "ssb_q43", "tpch_q7", "tpch_q9", "tpch_q4", "tpch_q13",
      "tpch_q17", "tpch_q18", "tpch_q19", "tpch_q21"]


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q, qs=None, sf=None, copart=False, replicated=False):
    qs = QS if qs is None else qs
    sf = SF if sf is None else sf
    try:
        import torch
        import torch.distributed as dist

        import hqgen
        from paper_conf_sigmod_funkebnmt18_b200 import hq
        from paper_conf_sigmod_funkebnmt18_b200.dist import DistributedEngine, partition, run_query
        from paper_conf_sigmod_funkebnmt18_b200.queries import QUERIES, load_tables

        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        torch.cuda.set_device(0)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        ctx = hq.Context(0)
        out = {}
        for qn in qs:
            qq = QUERIES[qn]
            n = hqgen.table_rows(qq.fact, sf)
            if copart:  # orders + lineitem co-partitioned by order, every rank builds locally
                crng, rng = hqgen.copartition(qq.fact, qq.copart, sf, rank, world)
                tables = load_tables(ctx, qq, sf, fact_range=rng, copart_range=crng)
            else:
                rng = partition(n, rank, world)
                tables = load_tables(ctx, qq, sf, fact_range=rng, skip_dims=rank != 0 and not replicated)
            E = DistributedEngine(ctx, tables, copartitioned=copart, replicated=replicated)
            r = run_query(E, qq)
            out[qn] = (r.rows(), r.qualifying) if r is not None else None
        q.put(("ok", rank, out))
        dist.barrier()
        dist.destroy_process_group()
    except Exception as e:  # pragma: no cover
        import traceback
        q.put(("err", rank, traceback.format_exc()))


def test_two_ranks_on_one_device_match_oracle():
    import hqgen
    import oracle
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    outs = [q.get(timeout=600) for _ in procs]
    for p in procs:
        p.join(timeout=120)
    errs = [o for o in outs if o[0] != "ok"]
    if errs:
        pytest.fail("\n\n".join(f"rank {o[1]}:\n{o[2]}" for o in errs))
    root = {k: v[0] for k, v in next(o[2] for o in outs if o[1] == 0).items()}
    ssb = {t: hqgen.generate(t, SF) for t in hqgen.SSB_TABLES}
    tpch = {t: hqgen.generate(t, SF) for t in hqgen.TPCH_TABLES}
    exp = {
        "ssb_q41": oracle.ssb_q41(ssb["lineorder"], ssb["date"], ssb["customer"], ssb["supplier"], ssb["part"]).rows(),
        "ssb_q31": oracle.ssb_q31(ssb["lineorder"], ssb["customer"], ssb["supplier"], ssb["date"]).rows(),
        "ssb_q11": oracle.ssb_q1(1, ssb["lineorder"], ssb["date"]).rows(),
        "tpch_q6": oracle.tpch_q6(tpch["lineitem"]).rows(),
        "tpch_q5": oracle.tpch_q5(tpch["tpch_customer"], tpch["orders"], tpch["lineitem"], tpch["tpch_supplier"],
                                  tpch["nation"], tpch["region"]).rows(),
        "tpch_q4": oracle.tpch_q4(tpch["orders"], tpch["lineitem"]).rows(),
        "tpch_q13": oracle.tpch_q13(tpch["tpch_customer"], tpch["orders"]).rows(),
        "tpch_q17": oracle.tpch_q17(tpch["tpch_part"], tpch["lineitem"]).rows(),
        "tpch_q18": oracle.tpch_q18(tpch["tpch_customer"], tpch["orders"], tpch["lineitem"]).rows(
            ["o_orderkey", "c_custkey", "o_orderdate", "o_totalprice", "sum_qty", "count"])[:100],
        "tpch_q19": oracle.tpch_q19(tpch["tpch_part"], tpch["lineitem"]).rows(),
        "tpch_q21": oracle.tpch_q21(tpch["tpch_supplier"], tpch["orders"], tpch["lineitem"], tpch["nation"]).rows()[:100],
        "tpch_q9": oracle.tpch_q9(tpch["tpch_part"], tpch["tpch_supplier"], tpch["lineitem"], tpch["partsupp"],
                                  tpch["orders"], tpch["nation"]).rows(),
        "tpch_q7": oracle.tpch_q7(tpch["tpch_customer"], tpch["orders"], tpch["lineitem"], tpch["tpch_supplier"],
                                  tpch["nation"]).rows(),
        "ssb_q43": oracle.ssb_q4(3, ssb["lineorder"], ssb["date"], ssb["customer"], ssb["supplier"], ssb["part"]).rows(),
    }
    for qn, rows in exp.items():
        assert root[qn] == rows, qn
    o1 = oracle.tpch_q1(tpch["lineitem"])
    got = [r[:6] + (r[9],) for r in root["tpch_q1"]]  # keys, 4 sums, count (AVG columns checked below)
    assert got == o1.rows(["l_returnflag", "l_linestatus", "sum_qty", "sum_base_price", "sum_disc_price",
                           "sum_charge", "count_order"])
    for r, avg in zip(root["tpch_q1"], o1.rows(["avg_qty", "avg_price", "avg_disc"])):
        assert all(abs(a - b) <= 1e-9 * abs(b) for a, b in zip(r[6:9], avg))
    # hash group-by (l_orderkey): ranks' groups all-gathered and merged on the root, then top 10
    o3 = oracle.tpch_q3(tpch["tpch_customer"], tpch["orders"], tpch["lineitem"])
    assert root["tpch_q3"] == o3.rows(["l_orderkey", "o_orderdate", "o_shippriority", "revenue", "count"])[:10]


F3 = ["tpch_q4", "tpch_q13", "tpch_q17", "tpch_q18", "tpch_q19", "tpch_q21"]


def test_two_ranks_tpch_multi_pipeline_sf1():
    """The multi-pipeline TPC-H plans at SF 1 (non-empty Q17/Q18/Q19 results) over two
    ranks: intermediate GROUP BYs over the lineitem / orders partitions are gathered and
    merged on the root (orders split by the range partition are combined), their builds
    broadcast, and the root finishes; the root's rows equal the oracle's."""
    import hqgen
    import oracle
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q, F3, 1.0)) for r in range(2)]
    for p in procs:
        p.start()
    outs = [q.get(timeout=900) for _ in procs]
    for p in procs:
        p.join(timeout=120)
    errs = [o for o in outs if o[0] != "ok"]
    if errs:
        pytest.fail("\n\n".join(f"rank {o[1]}:\n{o[2]}" for o in errs))
    root = {k: v[0] for k, v in next(o[2] for o in outs if o[1] == 0).items()}
    assert all(o[2][qn] is None for o in outs if o[1] != 0 for qn in F3)
    t = {x: hqgen.generate(x, 1.0) for x in hqgen.TPCH_TABLES}
    exp = {
        "tpch_q4": oracle.tpch_q4(t["orders"], t["lineitem"]).rows(),
        "tpch_q13": oracle.tpch_q13(t["tpch_customer"], t["orders"]).rows(),
        "tpch_q17": oracle.tpch_q17(t["tpch_part"], t["lineitem"]).rows(),
        "tpch_q18": oracle.tpch_q18(t["tpch_customer"], t["orders"], t["lineitem"]).rows(
            ["o_orderkey", "c_custkey", "o_orderdate", "o_totalprice", "sum_qty", "count"])[:100],
        "tpch_q19": oracle.tpch_q19(t["tpch_part"], t["lineitem"]).rows(),
        "tpch_q21": oracle.tpch_q21(t["tpch_supplier"], t["orders"], t["lineitem"], t["nation"]).rows()[:100],
    }
    for qn, rows in exp.items():
        assert root[qn] == rows, qn
        assert len(rows) > 0, qn


@pytest.mark.parametrize("world,sf", [(2, 0.01), (3, 1.0)])
def test_copartitioned_tpch_q3(world, sf):
    """TPC-H Q3 with orders and lineitem co-partitioned by order (hqgen.copartition):
    every rank builds its customer / orders tables locally (no broadcast), runs its
    ORDER BY / LIMIT over its own (disjoint) orderkey groups, and the root merges the
    ranks' top rows; rows and the qualifying count equal the oracle's."""
    import hqgen
    import oracle
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q, ["tpch_q3"], sf, True)) for r in range(world)]
    for p in procs:
        p.start()
    outs = [q.get(timeout=900) for _ in procs]
    for p in procs:
        p.join(timeout=120)
    errs = [o for o in outs if o[0] != "ok"]
    if errs:
        pytest.fail("\n\n".join(f"rank {o[1]}:\n{o[2]}" for o in errs))
    rows, qual = next(o[2] for o in outs if o[1] == 0)["tpch_q3"]
    assert all(o[2]["tpch_q3"] is None for o in outs if o[1] != 0)
    t = {x: hqgen.generate(x, sf) for x in ("tpch_customer", "orders", "lineitem")}
    o3 = oracle.tpch_q3(t["tpch_customer"], t["orders"], t["lineitem"])
    assert rows == o3.rows(["l_orderkey", "o_orderdate", "o_shippriority", "revenue", "count"])[:10]
    assert qual == int(o3.columns["count"].sum())  # lineitem rows that reached the GROUP BY, all ranks


REPL = ["ssb_q41", "ssb_q31", "tpch_q1", "tpch_q3", "tpch_q5", "tpch_q4", "tpch_q13", "tpch_q18", "tpch_q21"]


def test_replicated_dimensions_match_oracle():
    """Replicated dimensions (the bench's default multi-GPU mode): every rank builds the
    dimension tables and runs the build-side pipelines itself (no broadcast), only
    tables over a gathered result are sent; two ranks at SF 0.01, rows equal the oracle."""
    import hqgen
    import oracle
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q, REPL, 0.01, False, True)) for r in range(2)]
    for p in procs:
        p.start()
    outs = [q.get(timeout=900) for _ in procs]
    for p in procs:
        p.join(timeout=120)
    errs = [o for o in outs if o[0] != "ok"]
    if errs:
        pytest.fail("\n\n".join(f"rank {o[1]}:\n{o[2]}" for o in errs))
    root = {k: v[0] for k, v in next(o[2] for o in outs if o[1] == 0).items()}
    assert all(o[2][qn] is None for o in outs if o[1] != 0 for qn in REPL)
    ssb = {t: hqgen.generate(t, 0.01) for t in hqgen.SSB_TABLES}
    t = {x: hqgen.generate(x, 0.01) for x in hqgen.TPCH_TABLES}
    exp = {
        "ssb_q41": oracle.ssb_q41(ssb["lineorder"], ssb["date"], ssb["customer"], ssb["supplier"], ssb["part"]).rows(),
        "ssb_q31": oracle.ssb_q31(ssb["lineorder"], ssb["customer"], ssb["supplier"], ssb["date"]).rows(),
        "tpch_q5": oracle.tpch_q5(t["tpch_customer"], t["orders"], t["lineitem"], t["tpch_supplier"], t["nation"],
                                  t["region"]).rows(),
        "tpch_q4": oracle.tpch_q4(t["orders"], t["lineitem"]).rows(),
        "tpch_q13": oracle.tpch_q13(t["tpch_customer"], t["orders"]).rows(),
        "tpch_q18": oracle.tpch_q18(t["tpch_customer"], t["orders"], t["lineitem"]).rows(
            ["o_orderkey", "c_custkey", "o_orderdate", "o_totalprice", "sum_qty", "count"])[:100],
        "tpch_q21": oracle.tpch_q21(t["tpch_supplier"], t["orders"], t["lineitem"], t["nation"]).rows()[:100],
    }
    for qn, rows in exp.items():
        assert root[qn] == rows, qn
    o3 = oracle.tpch_q3(t["tpch_customer"], t["orders"], t["lineitem"])
    assert root["tpch_q3"] == o3.rows(["l_orderkey", "o_orderdate", "o_shippriority", "revenue", "count"])[:10]
    o1 = oracle.tpch_q1(t["lineitem"])
    assert [r[:6] + (r[9],) for r in root["tpch_q1"]] == o1.rows(
        ["l_returnflag", "l_linestatus", "sum_qty", "sum_base_price", "sum_disc_price", "sum_charge", "count_order"])


@pytest.mark.parametrize("replicated", [False, True])
def test_two_ranks_materialise_gathers_rows(replicated):
    """A partitioned materialising pipeline (SSB Q3.1 materialised, SURVEY §8(e)
    "materialise sinks"): each rank's rows are all-gathered to the root; the root's rows
    (sorted) and qualifying count equal the oracle's on the whole table."""
    import hqgen
    import oracle
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q, ["ssb_q31_mat"], 0.01, False, replicated))
             for r in range(2)]
    for p in procs:
        p.start()
    outs = [q.get(timeout=600) for _ in procs]
    for p in procs:
        p.join(timeout=120)
    errs = [o for o in outs if o[0] != "ok"]
    if errs:
        pytest.fail("\n\n".join(f"rank {o[1]}:\n{o[2]}" for o in errs))
    rows, qual = next(o[2] for o in outs if o[1] == 0)["ssb_q31_mat"]
    ssb = {t: hqgen.generate(t, 0.01) for t in hqgen.SSB_TABLES}
    o = oracle.ssb_q31_mat(ssb["lineorder"], ssb["customer"], ssb["supplier"], ssb["date"])
    assert sorted(rows) == o.rows()
    assert qual == o.nrows


def _prepared_worker(rank, world, port, q, qs, sf):
    try:
        import torch
        import torch.distributed as dist

        import hqgen
        from paper_conf_sigmod_funkebnmt18_b200 import hq
        from paper_conf_sigmod_funkebnmt18_b200.dist import DistributedEngine, partition
        from paper_conf_sigmod_funkebnmt18_b200.queries import QUERIES, load_tables

        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        torch.cuda.set_device(0)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        ctx = hq.Context(0)
        out = {}
        for qn in qs:
            qq = QUERIES[qn]
            rng = partition(hqgen.table_rows(qq.fact, sf), rank, world)
            E = DistributedEngine(ctx, load_tables(ctx, qq, sf, fact_range=rng), replicated=True)
            pq = E.prepare(qq)
            runs = [pq.execute() for _ in range(3)]
            pq.close()
            out[qn] = [r.rows() if r is not None else None for r in runs]
        q.put(("ok", rank, out))
        dist.barrier()
        dist.destroy_process_group()
    except Exception:  # pragma: no cover
        import traceback
        q.put(("err", rank, traceback.format_exc()))


def test_prepared_distributed_step_matches_oracle():
    """dist.PreparedDistQuery: graph A (builds, pipeline, [partials | faults] packed),
    the all-reduce between the graphs, graph B (copy-back, finalize) -- three launches per
    query over two ranks, every launch's root rows equal the oracle."""
    import hqgen
    import oracle
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    qs = ["ssb_q41", "ssb_q31", "tpch_q6"]
    procs = [ctx.Process(target=_prepared_worker, args=(r, 2, port, q, qs, 0.01)) for r in range(2)]
    for p in procs:
        p.start()
    outs = [q.get(timeout=600) for _ in procs]
    for p in procs:
        p.join(timeout=120)
    errs = [o for o in outs if o[0] != "ok"]
    if errs:
        pytest.fail("\n\n".join(f"rank {o[1]}:\n{o[2]}" for o in errs))
    root = next(o[2] for o in outs if o[1] == 0)
    assert all(r is None for o in outs if o[1] != 0 for qn in qs for r in o[2][qn])
    ssb = {t: hqgen.generate(t, 0.01) for t in hqgen.SSB_TABLES}
    li = hqgen.generate("lineitem", 0.01)
    exp = {"ssb_q41": oracle.ssb_q41(ssb["lineorder"], ssb["date"], ssb["customer"], ssb["supplier"], ssb["part"]).rows(),
           "ssb_q31": oracle.ssb_q31(ssb["lineorder"], ssb["customer"], ssb["supplier"], ssb["date"]).rows(),
           "tpch_q6": oracle.tpch_q6(li).rows()}
    for qn in qs:
        for rows in root[qn]:
            assert rows == exp[qn], qn
