"""Plan construction and single-device query execution on top of libhq.

A query is a sequence of *fusion operators* (§4.1):
hash builds (pipeline breakers) followed by probe pipelines, each pipeline one
``hq_run_pipeline`` call = one fused kernel.  ``PlanBuilder`` fills the
``hq_plan`` descriptor (plans given explicitly with their fusion
operators), ``Engine`` owns the device tables and runs builds and pipelines.
``dist.DistributedEngine`` overrides builds (root builds + NCCL broadcast) and
the final reduce.
"""
from __future__ import annotations

from dataclasses import dataclass, field
from typing import Dict, List, Optional, Sequence, Tuple

import numpy as np

from . import hq

_OPC = {"load": hq.I_LOAD, "add": hq.I_ADD, "sub": hq.I_SUB, "rsub": hq.I_RSUB, "mul": hq.I_MUL,
        "div": hq.I_DIV, "mod": hq.I_MOD, "and_eq": hq.I_AND_EQ, "and_ne": hq.I_AND_NE, "and_lt": hq.I_AND_LT,
        "and_le": hq.I_AND_LE, "and_gt": hq.I_AND_GT, "and_ge": hq.I_AND_GE, "and_in": hq.I_AND_IN, "or": hq.I_OR}
_AGG = {"sum": hq.AGG_SUM, "count": hq.AGG_COUNT, "min": hq.AGG_MIN, "max": hq.AGG_MAX, "avg": hq.AGG_AVG}
_TYPES = {"i8": hq.HQ_I8, "i32": hq.HQ_I32, "i64": hq.HQ_I64}


class PlanBuilder:
    """Builds one hq_plan over a fact table.  Registers are named: fact column
    names, and temporaries created by probe payloads / compute ops."""

    def __init__(self, fact: hq.Table):
        self.fact = fact
        self.plan = hq.Plan()
        self.plan.fact = fact.h
        self.plan.row_begin = 0
        self.plan.row_end = -1
        self.tmps: Dict[str, int] = {}
        self.keep: List[object] = [fact]
        self.result_names: List[str] = []

    # registers
    def reg(self, name: str) -> int:
        if name in self.tmps:
            return self.tmps[name]
        return self.fact.col(name)

    def _new_tmp(self, name: str) -> int:
        if name in self.tmps:
            return self.tmps[name]
        if len(self.tmps) >= hq.MAX_TMP:
            raise ValueError("too many temporaries")
        self.tmps[name] = hq.TMP(len(self.tmps))
        return self.tmps[name]

    def _op(self) -> hq.Op:
        if self.plan.nops >= hq.MAX_OPS:
            raise ValueError("too many ops")
        op = self.plan.ops[self.plan.nops]
        self.plan.nops += 1
        return op

    # operators
    def filter(self, col: str, cmp, lo=0, hi=0) -> "PlanBuilder":
        op = self._op()
        op.kind = hq.OP_FILTER
        op.filter = hq.make_pred(self.reg(col), cmp, lo, hi)
        return self

    def probe(self, ht: hq.Hash, key: str, mode: str = "inner", payload: Sequence[str] = (),
              key2: Optional[str] = None) -> "PlanBuilder":
        """key2: the second key register of a composite (two-column) join key."""
        op = self._op()
        op.kind = hq.OP_PROBE
        op.ht = ht.h
        op.key_reg = self.reg(key)
        if key2 is not None:
            op.key2_reg = self.reg(key2)
        op.mode = {"inner": hq.PROBE_INNER, "semi": hq.PROBE_SEMI, "anti": hq.PROBE_ANTI, "outer": hq.PROBE_OUTER}[mode]
        op.npayload = len(payload)
        for i, name in enumerate(payload):
            op.payload_dst[i] = self._new_tmp(name)
        self.keep.append(ht)
        return self

    def compute(self, dst: str, code: Sequence[Tuple[str, object]]) -> "PlanBuilder":
        """code: accumulator-machine program, e.g. [("load","a"), ("rsub",100), ("mul","b")].
        Predicate instructions name a register and a constant: ("and_le", "p_size", 5),
        ("and_in", "p_container", [codes...]) (a conjunction; "or" joins a predicate temp)."""
        op = self._op()
        op.kind = hq.OP_COMPUTE
        if len(code) > hq.MAX_INSN:
            raise ValueError("expression too long")
        op.ninsn = len(code)
        for i, (opc, arg, *const) in enumerate(code):
            ins = op.code[i]
            ins.opc = _OPC[opc]
            if const:  # predicate instruction: register arg, constant (or IN-list) const[0]
                c = const[0]
                if opc == "and_in":
                    m = 0
                    for v in c:
                        if not 0 <= int(v) < 64:
                            raise ValueError("and_in values must be codes 0..63")
                        m |= 1 << int(v)
                    c = m - (1 << 64) if m >= (1 << 63) else m
                ins.reg = self.reg(arg)
                ins.imm = int(c)
            elif isinstance(arg, str):
                ins.reg = self.reg(arg)
            else:
                ins.reg = -1
                ins.imm = int(arg)
        op.dst = self._new_tmp(dst)
        return self

    # sinks
    def aggregate(self, keys: Sequence[Tuple[str, int, int]] = (), aggs: Sequence[Tuple] = (),
                  order: Sequence[Tuple[str, bool]] = (), limit: int = 0, group_capacity: int = 0,
                  agg_names: Sequence[str] = ()) -> "PlanBuilder":
        """keys: (register, min, cardinality); aggs: (fn, register|None[, scale]);
        order: (result column name, descending); result columns = keys then aggs."""
        P = self.plan
        P.sink = hq.SINK_AGG
        P.nkeys = len(keys)
        for i, (name, mn, card) in enumerate(keys):
            P.key_reg[i] = self.reg(name)
            P.key_min[i] = int(mn)
            P.key_card[i] = int(card)
        P.naggs = len(aggs)
        for i, a in enumerate(aggs):
            fn, name = a[0], a[1]
            P.agg_fn[i] = _AGG[fn]
            P.agg_reg[i] = self.reg(name) if name is not None else 0
            P.agg_scale[i] = a[2] if len(a) > 2 else 0
        P.group_capacity = int(group_capacity)
        names = [k[0] for k in keys] + list(agg_names or [f"{a[0]}_{a[1]}" for a in aggs])
        self.result_names = names
        P.norder = len(order)
        for i, (name, desc) in enumerate(order):
            P.order_col[i] = names.index(name)
            P.order_desc[i] = int(bool(desc))
        P.limit = int(limit)
        return self

    def materialise(self, outs: Sequence[Tuple[str, str]], capacity: int = 0,
                    names: Sequence[str] = ()) -> "PlanBuilder":
        P = self.plan
        P.sink = hq.SINK_MATERIALISE
        P.nout = len(outs)
        for i, (name, t) in enumerate(outs):
            P.out_reg[i] = self.reg(name)
            P.out_type[i] = _TYPES[t]
        P.capacity = int(capacity)
        self.result_names = list(names or [o[0] for o in outs])
        return self


@dataclass
class QueryResult:
    """Fetched result: named numpy columns (sorted/limited as the plan says)."""
    columns: Dict[str, np.ndarray] = field(default_factory=dict)
    qualifying: int = 0

    @property
    def nrows(self) -> int:
        return len(next(iter(self.columns.values()))) if self.columns else 0

    def rows(self, names: Optional[List[str]] = None) -> List[tuple]:
        names = names or list(self.columns)
        return list(zip(*[self.columns[n].tolist() for n in names]))


def fetch(res: hq.Result, names: Sequence[str]) -> QueryResult:
    cols = res.fetch()
    return QueryResult({n: c for n, c in zip(names, cols)}, res.qualifying())


class Engine:
    """Single-device execution: device tables by name, builds and pipelines.

    exec_mode: hq.EXEC_FUSED (the compound kernel) or hq.EXEC_OAAT
    (operator-at-a-time baseline of the same plan).  resolution: hq.RES_LRGP or
    hq.RES_ATOMIC (ablation).  fact_range: optional (begin, end) rows of the
    fact table for partitioned pipelines (logical partitions on one device).
    """

    def __init__(self, ctx: hq.Context, tables: Dict[str, hq.Table], exec_mode: int = hq.EXEC_FUSED,
                 resolution: int = hq.RES_LRGP, fact_range: Optional[Tuple[int, int]] = None,
                 stream_block: Optional[int] = None):
        self.ctx = ctx
        self.tables = tables
        self.exec_mode = exec_mode
        self.resolution = resolution
        self.fact_range = fact_range
        self.stream_block = stream_block  # rows per block for host-streamed fact tables

    def table(self, name: str) -> hq.Table:
        return self.tables[name]

    #: whether this engine runs build-side (unpartitioned) pipelines; False on
    #: the non-root ranks of a DistributedEngine
    builds_here = True

    def plan(self, fact: str) -> PlanBuilder:
        return PlanBuilder(self.tables[fact])

    def plan_over(self, res: hq.Result, names: Sequence[str]) -> PlanBuilder:
        """A pipeline over a finalized aggregation (or materialised) result, e.g. the
        outer GROUP BY of TPC-H Q13 or a HAVING / derived predicate; run it with
        partitioned=False."""
        pb = PlanBuilder(res.as_table(list(names)))
        pb.keep.append(res)
        return pb

    def hash(self, table: str, key: str, payload: Sequence[str] = (),
             preds: Sequence[Tuple] = (), expected_rows: int = 0, key2: Optional[str] = None) -> hq.Hash:
        """key2: second column of a composite join key (e.g. (ps_partkey, ps_suppkey))."""
        t = self.tables[table]
        ps = [hq.make_pred(t.col(p[0]), *p[1:]) for p in preds]
        return self.ctx.build_hash(t, t.col(key), [t.col(c) for c in payload], ps, expected_rows,
                                   None if key2 is None else t.col(key2))

    def hashes(self, specs: Sequence[dict]) -> List[hq.Hash]:
        """Independent builds (a query's dimension tables) with one host sync:
        specs = [dict(table=, key=, payload=(), preds=(), expected_rows=0), ...]."""
        out = []
        for sp in specs:
            t = self.tables[sp["table"]]
            ps = [hq.make_pred(t.col(p[0]), *p[1:]) for p in sp.get("preds", ())]
            k2 = sp.get("key2")
            out.append((t, t.col(sp["key"]), [t.col(c) for c in sp.get("payload", ())], ps, sp.get("expected_rows", 0),
                        None if k2 is None else t.col(k2)))
        return self.ctx.build_hashes(out)

    def hash_from(self, res: Optional[hq.Result], names: Sequence[str], key: str,
                  payload: Sequence[str] = (), preds: Sequence[Tuple] = ()) -> hq.Hash:
        """Build a hash table from a materialised (or aggregated) pipeline result
        (pipeline breaker); preds filter its rows (e.g. a HAVING clause)."""
        t = res.as_table(list(names))
        ps = [hq.make_pred(t.col(p[0]), *p[1:]) for p in preds]
        return self.ctx.build_hash(t, t.col(key), [t.col(c) for c in payload], ps)

    def run(self, pb: PlanBuilder, partitioned: bool = True) -> Optional[hq.Result]:
        P = pb.plan
        P.exec = self.exec_mode
        P.resolution = self.resolution
        if partitioned and self.fact_range is not None:
            P.row_begin, P.row_end = self.fact_range
        block = self.stream_block if getattr(pb.fact, "host_stream", False) else None
        return self.ctx.run(P, keep=pb.keep, block_rows=block)

    def finish(self, res: hq.Result, pb: PlanBuilder) -> QueryResult:
        return fetch(res, pb.result_names)

    def key_domain(self, table: str, col: str) -> Tuple[int, int]:
        """(min, cardinality) of a column, for declaring a tight GROUP BY key domain
        (lets libhq use a dense group table for large groupings, hq.h key_card)."""
        lo, hi = self.tables[table].column_range(col)
        return (0, 1) if lo > hi else (lo, hi - lo + 1)

    def prepare(self, query, **kw) -> "PreparedQuery":
        """A prepared query: executed once eagerly (kernels compiled, build statistics
        cached), then recorded into a CUDA graph whose launches re-run all its device work
        (hq.h "prepared queries").  Raises HQError(HQ_ERR_STATE) for queries that need
        the host mid-way (materialised intermediates, large results, ...)."""
        return PreparedQuery(self, query, **kw)

    def gather(self, res: Optional[hq.Result], pb: PlanBuilder) -> Optional[hq.Result]:
        """The complete result of a partitioned pipeline whose aggregation feeds a later
        build or pipeline (an intermediate GROUP BY): on one device, the result itself."""
        return res


class PreparedQuery:
    """One query step recorded as a CUDA graph (Engine.prepare).  execute() launches it:
    the hash builds, compound kernels and finalization all run again on the device;
    only the host-side planning was done once."""

    def __init__(self, E: Engine, query, **kw):
        self.E, self.query, self.kw = E, query, kw
        query.execute(E, **kw)  # eager run: JIT kernels compiled, build statistics cached
        ctx = E.ctx
        ctx.capture_begin()
        try:
            self.res, self.pb = query.run(E, **kw)
            self.res.finalize()
        except BaseException:
            ctx.capture_abort()
            raise
        self.graph = ctx.capture_end()

    def execute(self) -> QueryResult:
        self.graph.launch()
        return fetch(self.res, self.pb.result_names)

    def close(self) -> None:
        self.graph.free()
