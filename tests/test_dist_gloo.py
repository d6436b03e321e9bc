"""Multi-process orchestration on CPU (gloo, world_size 2): the same
range-partition / broadcast / reduce functions the NCCL path uses
(paper_conf_sigmod_funkebnmt18_b200.dist), with a TEST-ONLY numpy stand-in for
the device engine's partial aggregates.  Pins: the reduced partials of the two
ranks equal the oracle on the whole table; broadcast tables (metadata rows and
buffers) arrive intact for 0, 1 and 3 tables; a root-side build error makes every
rank raise."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import hqgen
from paper_conf_sigmod_funkebnmt18_b200 import hq
from paper_conf_sigmod_funkebnmt18_b200.dist import (RootError, broadcast_tables, meta_from_row, meta_row, partition,
                                                     reduce_partials)

SF = 0.01


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _q41_partials(lo, c, s, p, d):
    """Test-only stand-in for the fused kernel's dense partial table: [count, profit]
    per (d_year, c_nation) group, same layout as hq_result_partials_view."""
    creg = c["c_region"][lo["lo_custkey"] - 1]
    sreg = s["s_region"][lo["lo_suppkey"] - 1]
    pm = p["p_mfgr"][lo["lo_partkey"] - 1]
    m = (creg == 1) & (sreg == 1) & (pm <= 1)
    year = lo["lo_orderdate"][m] // 10000
    nat = c["c_nation"][lo["lo_custkey"][m] - 1].astype(np.int64)
    g = (year - 1992) * 25 + nat
    t = np.zeros((175, 2), np.int64)
    np.add.at(t[:, 0], g, 1)
    np.add.at(t[:, 1], g, lo["lo_revenue"][m].astype(np.int64) - lo["lo_supplycost"][m])
    return t


def _stub_meta(k, nbytes):
    """A hash-table metadata record with every field set (pay_set words with bit 63 on)."""
    m = hq.HashMeta()
    m.capacity, m.slot_words, m.npayload, m.nkeys = 1 << (10 + k), 2, 1, 1000 + k
    m.bytes, m.key_min, m.layout = nbytes, -5 - k, k % 2
    m.pay_min, m.pay_max, m.key_max = -3, 200 + k, 99999
    for i in range(4):
        m.pay_set[i] = (1 << 63) | (0x0123456789ABCDEF >> i) | k
    m.composite = k % 2
    m.compact_kind = k % 4
    return m


def _worker(rank, world, port, q):
    try:
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        n = hqgen.table_rows("lineorder", SF)
        a, b = partition(n, rank, world)
        lo = hqgen.generate("lineorder", SF, row_range=(a, b))
        dims = {t: hqgen.generate(t, SF) for t in ("customer", "supplier", "part", "date")}
        # root "builds" and broadcasts tables (the hash-table slot arrays on GPUs): n = 0, 1, 3
        blob = np.ascontiguousarray(dims["customer"]["c_custkey"][dims["customer"]["c_region"] == 1]).view(np.uint8)
        # with a shared receive-size state (the engine's): the first message grows it (two
        # collectives), repeated and smaller ones fit in one
        state = {}
        for nt, stateful in ((0, False), (1, False), (3, False), (1, True), (3, True), (3, True), (1, True),
                             (0, True)):
            blobs = [np.roll(blob, k + nt).copy() for k in range(nt)]
            metas = [_stub_meta(k, x.nbytes) for k, x in enumerate(blobs)]
            st = state if stateful else None
            if rank == 0:
                rows, bufs = broadcast_tables([meta_row(m) for m in metas], [torch.from_numpy(x) for x in blobs], nt, 0,
                                              "cpu", state=st)
            else:
                rows, bufs = broadcast_tables(None, None, nt, 0, "cpu", state=st)
            assert len(rows) == len(bufs) == nt
            for m, r, buf, ref in zip(metas, rows, bufs, blobs):
                got = meta_from_row(r)
                assert bytes(got) == bytes(m)  # every field, pay_set bit 63 included
                assert np.array_equal(buf.numpy(), ref)
        # a root-side build error: the root re-raises it, the other rank raises RootError
        if rank == 0:
            try:
                broadcast_tables(None, None, 2, 0, "cpu", err=hq.HQError(hq.HQ_ERR_DUP_KEY, "dup"), state=state)
                raise AssertionError("root did not re-raise")
            except hq.HQError as e:
                assert e.code == hq.HQ_ERR_DUP_KEY and not isinstance(e, RootError)
        else:
            try:
                broadcast_tables(None, None, 2, 0, "cpu", state=state)
                raise AssertionError("rank 1 did not raise")
            except RootError as e:
                assert e.code == hq.HQ_ERR_DUP_KEY
        part = torch.from_numpy(_q41_partials(lo, dims["customer"], dims["supplier"], dims["part"], dims["date"]).ravel().copy())
        reduce_partials(part, 0)
        if rank == 0:
            q.put(("ok", part.numpy().reshape(175, 2), (a, b)))
        else:
            q.put(("ok", None, (a, b)))
        dist.barrier()
        dist.destroy_process_group()
    except Exception as e:  # pragma: no cover
        q.put(("err", repr(e), None))


def test_partition_covers_range():
    for n in (0, 1, 7, 1000, 600_037_902):
        for w in (1, 2, 3, 8):
            parts = [partition(n, r, w) for r in range(w)]
            assert parts[0][0] == 0 and parts[-1][1] == n
            assert all(parts[i][1] == parts[i + 1][0] for i in range(w - 1))


def test_two_rank_reduce_matches_oracle():
    import oracle
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    outs = [q.get(timeout=240) for _ in procs]
    for p in procs:
        p.join(timeout=60)
    assert all(o[0] == "ok" for o in outs), outs
    table = next(o[1] for o in outs if o[1] is not None)
    ranges = sorted(o[2] for o in outs)
    assert ranges[0][0] == 0 and ranges[0][1] == ranges[1][0]
    ssb = {t: hqgen.generate(t, SF) for t in hqgen.SSB_TABLES}
    ref = oracle.ssb_q41(ssb["lineorder"], ssb["date"], ssb["customer"], ssb["supplier"], ssb["part"])
    got = [(1992 + g // 25, g % 25, int(table[g, 1]), int(table[g, 0])) for g in range(175) if table[g, 0] > 0]
    assert got == ref.rows()
