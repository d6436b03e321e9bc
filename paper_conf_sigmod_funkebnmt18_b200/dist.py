"""Multi-GPU orchestration: one process per GPU.

* the fact table is range-partitioned: rank r owns rows [r*N/P, (r+1)*N/P);
  the generator is partition-invariant, so the union equals the P=1 input;
* dimension hash tables are built once on the root and broadcast as raw slot
  arrays (``hq_hash_device_view`` -> ``dist.broadcast`` over NCCL/NVLink ->
  ``hq_hash_import``); build-side pipelines (e.g. TPC-H Q3's orders side) run
  on the root only;
* each rank runs the fused pipeline over its range; dense partial aggregates
  ([count, agg...] per group, int64) are combined with ONE ``dist.reduce``
  (SUM) to the root, which finalizes (ORDER BY / LIMIT on GPU 0).

The collectives here are backend-agnostic torch.distributed calls (NCCL on the
GPUs; the CPU tests drive the same functions with gloo and a test-only
stand-in for the device engine).  The paper itself is single-device; this is
new (north_star).
"""
from __future__ import annotations

import os
import sys
from typing import List, Optional, Sequence, Tuple

import torch
import torch.distributed as dist

from . import hq
from .engine import Engine, PlanBuilder, QueryResult, fetch


def partition(n: int, rank: int, world: int) -> Tuple[int, int]:
    """Row range of `rank` in a range partition of n rows over `world` ranks."""
    return n * rank // world, n * (rank + 1) // world


def _i64(u: int) -> int:
    """uint64 bit pattern as a signed int64 (torch.int64 transport)."""
    return u - (1 << 64) if u >= (1 << 63) else u


# hq_hash_meta <-> one int64 row of the metadata broadcast
META_COLS = 16


def meta_row(m: hq.HashMeta) -> List[int]:
    return ([m.capacity, m.slot_words, m.npayload, m.nkeys, m.bytes, m.key_min, m.layout, m.pay_min, m.pay_max,
             m.key_max] + [_i64(w) for w in m.pay_set] + [m.composite, m.compact_kind])


def meta_from_row(r: Sequence[int]) -> hq.HashMeta:
    hm = hq.HashMeta()
    (hm.capacity, hm.slot_words, hm.npayload, hm.nkeys, hm.bytes, hm.key_min, hm.layout,
     hm.pay_min, hm.pay_max, hm.key_max) = [int(x) for x in r[:10]]
    for k in range(4):
        hm.pay_set[k] = int(r[10 + k]) & 0xFFFFFFFFFFFFFFFF
    hm.composite = int(r[14])
    hm.compact_kind = int(r[15])
    return hm


class RootError(hq.HQError):
    """Raised on the ranks that did not fail when the root's build (or another rank's
    pipeline) did: every rank raises, none is left waiting in a collective."""


def _offsets(rows: Sequence[Sequence[int]]) -> Tuple[List[int], int]:
    """Byte offsets of the tables' slot arrays in the packed broadcast buffer (256-B aligned)."""
    offs, tot = [], 0
    for r in rows:
        offs.append(tot)
        tot += (int(r[4]) + 255) // 256 * 256
    return offs, tot


def broadcast_tables(rows: Optional[List[List[int]]], bufs: Optional[List[torch.Tensor]], n: int, root: int,
                     device, err: Optional[BaseException] = None) -> Tuple[List[List[int]], List[torch.Tensor]]:
    """Broadcast n root-built tables with TWO collectives: an (n+1) x 16 int64 metadata
    block (row n = the root's status: error code or 0), then ONE byte buffer holding every
    slot array at 256-B aligned offsets (the root packs them with device copies; the
    other ranks get views into it).  Root: rows / bufs given; other ranks: None.  A
    root-side error is broadcast before the root re-raises it, so the other ranks raise
    RootError instead of blocking in the next collective."""
    rank = dist.get_rank()
    meta = torch.zeros((n + 1, META_COLS), dtype=torch.int64, device=device)
    if rank == root:
        if err is not None:
            meta[n, 0] = getattr(err, "code", hq.HQ_ERR_STATE) or hq.HQ_ERR_STATE
        elif n:
            meta[:n] = torch.tensor(rows, dtype=torch.int64)
    dist.broadcast(meta, src=root)
    if rank == root:
        if err is not None:
            raise err
        if n == 0:
            return rows, bufs
        offs, tot = _offsets(rows)
        packed = torch.empty(tot, dtype=torch.uint8, device=device)
        for o, b in zip(offs, bufs):
            packed[o:o + b.numel()].copy_(b)
        dist.broadcast(packed, src=root)
        return rows, bufs
    m = meta.cpu().tolist()
    if m[n][0] != 0:
        raise RootError(int(m[n][0]), "hash build failed on the root rank")
    rows = m[:n]
    if n == 0:
        return rows, []
    offs, tot = _offsets(rows)
    packed = torch.empty(tot, dtype=torch.uint8, device=device)
    dist.broadcast(packed, src=root)
    return rows, [packed[o:o + int(r[4])] for o, r in zip(offs, rows)]


def reduce_partials(t: torch.Tensor, root: int) -> None:
    """Exact integer SUM of the ranks' partial aggregates (one all-reduce: NCCL
    over NVLink on the GPUs; gloo in the CPU tests).  Only the root finalizes."""
    dist.all_reduce(t, op=dist.ReduceOp.SUM)


class _CudaView:
    """Zero-copy torch view of a library-owned device buffer."""

    def __init__(self, ptr: int, n: int, typestr: str):
        self.__cuda_array_interface__ = {"shape": (n,), "typestr": typestr, "data": (ptr, False), "version": 3}


def device_view(ptr: int, nbytes: int, dtype=torch.uint8) -> torch.Tensor:
    typestr = {torch.uint8: "|u1", torch.int64: "<i8"}[dtype]
    n = nbytes // (1 if dtype == torch.uint8 else 8)
    return torch.as_tensor(_CudaView(ptr, n, typestr), device="cuda")


class DistributedEngine(Engine):
    """Engine whose builds happen on the root and are broadcast, and whose
    partitioned pipelines end with one reduce of the dense partials."""

    def __init__(self, ctx: hq.Context, tables, root: int = 0, **kw):
        super().__init__(ctx, tables, **kw)
        self.rank = dist.get_rank()
        self.world = dist.get_world_size()
        self.root = root
        self.device = torch.device("cuda", ctx.device)
        self._built: List[hq.Hash] = []
        self.builds_here = self.rank == root
        # HQ_DIST_FAULT_TRACE=1 (debug): re-read every root build's fault word after the
        # final fetch and report the ones that changed since the build
        self._trace: Optional[List[Tuple[str, hq.Hash, List[int]]]] = (
            [] if os.environ.get("HQ_DIST_FAULT_TRACE") == "1" else None)

    def _share_many(self, hs: Optional[Sequence[hq.Hash]], n: int, err: Optional[BaseException] = None) -> List[hq.Hash]:
        """Broadcast n root-built tables (broadcast_tables: one metadata broadcast, one
        asynchronous broadcast per slot array, no host read on the root) and import them
        on the other ranks.  Build faults are not read here (that would sync per table):
        the root's fault words travel with the pipeline's reduce (_reduce_checked)."""
        if self.rank == self.root:
            rows, views = [], []
            if err is None:
                for h in hs:
                    ptr, m = h.device_view()
                    self._built.append(h)
                    if self._trace is not None:
                        self._trace.append((f"build#{len(self._trace)} rows={m.nkeys} cap={m.capacity}", h,
                                            self._faults_of(h)))
                    views.append(device_view(ptr, int(m.bytes)))
                    rows.append(meta_row(m))
            broadcast_tables(rows, views, n, self.root, self.device, err)
            return list(hs)
        rows, bufs = broadcast_tables(None, None, n, self.root, self.device)
        return [self.ctx.import_hash(meta_from_row(r), b.data_ptr(), keep=b) for r, b in zip(rows, bufs)]  # views keep the buffer

    def _root_build(self, fn, n: int):
        hs, err = None, None
        if self.rank == self.root:
            try:
                hs = fn()
            except hq.HQError as e:
                err = e
        return self._share_many(hs, n, err)

    def hash(self, table, key, payload=(), preds=(), expected_rows=0, key2=None) -> hq.Hash:
        return self._root_build(lambda: [super(DistributedEngine, self).hash(table, key, payload, preds,
                                                                             expected_rows, key2)], 1)[0]

    def hashes(self, specs) -> List[hq.Hash]:
        return self._root_build(lambda: super(DistributedEngine, self).hashes(specs), len(specs))

    def hash_from(self, res, names, key, payload=(), preds=()) -> hq.Hash:
        return self._root_build(lambda: [super(DistributedEngine, self).hash_from(res, names, key, payload,
                                                                                  preds)], 1)[0]

    @staticmethod
    def _hash_grouped(P: hq.Plan) -> bool:
        if P.sink != hq.SINK_AGG or P.nkeys == 0:
            return False
        prod = 1
        for i in range(P.nkeys):
            prod *= P.key_card[i]
        if any(P.agg_fn[a] in (hq.AGG_MIN, hq.AGG_MAX) for a in range(P.naggs)):
            return True  # MIN / MAX partials do not combine with a SUM all-reduce: merge the groups
        return prod > 65536  # libhq's dense/hash switch (hqk::DENSE_LIMIT)

    def run(self, pb: PlanBuilder, partitioned: bool = True) -> Optional[hq.Result]:
        if not partitioned:
            pb.root_only = True  # a build-side or post-merge pipeline: the root's result is complete
            if self.rank != self.root:
                return None
            return super().run(pb, partitioned)
        P = pb.plan
        if partitioned and self._hash_grouped(P):
            # ranks keep all their groups; ORDER BY / LIMIT run after the root's merge
            pb.dist_order = ([(P.order_col[i], P.order_desc[i]) for i in range(P.norder)], P.limit)
            P.norder, P.limit = 0, 0
        return super().run(pb, partitioned)

    def _faults_of(self, h: hq.Hash) -> List[int]:
        st = torch.zeros(hq.FAULT_WORDS, dtype=torch.int64, device=self.device)
        self.ctx.gather_faults([h], [], st.data_ptr())
        return st.tolist()

    def _trace_report(self, where: str) -> None:
        if not self._trace:
            return
        for label, h, before in self._trace:
            now = self._faults_of(h)
            if now != before:
                print(f"[hq dist trace] rank {self.rank} {where}: {label} fault words {before} -> {now}",
                      file=sys.stderr, flush=True)
            try:  # the syncing check round 1 ran here (hq_hash_info)
                h.info()
            except hq.HQError as e:
                print(f"[hq dist trace] rank {self.rank} {where}: {label} hq_hash_info raised {e}", file=sys.stderr,
                      flush=True)
        self._trace.clear()

    def _reduce_checked(self, res: hq.Result) -> None:
        """ONE all-reduce of [dense partials | fault words]: the partials are summed
        (exact int64), and the fault words -- the root's build faults and every rank's
        pipeline faults, gathered on the device (hq_gather_faults) -- are summed too, so
        every rank sees every rank's faults and raises, or none does.  One host read of
        the 32 fault words at the end; no per-table synchronisation."""
        ptr, nbytes = res.partials_view()
        n = nbytes // 8
        red = torch.empty(n + hq.FAULT_WORDS, dtype=torch.int64, device=self.device)
        red[:n].copy_(device_view(ptr, nbytes, torch.int64))
        built, self._built = self._built, []
        self.ctx.gather_faults(built, [res], red.data_ptr() + n * 8)
        reduce_partials(red, self.root)
        res.from_partials(red.data_ptr(), nbytes)
        hq.raise_faults(red[n:].tolist())

    def _root_only_checked(self, res: Optional[hq.Result]) -> None:
        """A root-only final pipeline: the root's build and pipeline faults are shared
        with one small all-reduce, so that all ranks raise together."""
        st = torch.zeros(hq.FAULT_WORDS, dtype=torch.int64, device=self.device)
        built, self._built = self._built, []
        if self.rank == self.root:
            self.ctx.gather_faults(built, [res] if res is not None else [], st.data_ptr())
        dist.all_reduce(st)
        hq.raise_faults(st.tolist())

    def finish(self, res: hq.Result, pb: PlanBuilder) -> Optional[QueryResult]:
        """Dense aggregates: one all-reduce of the partials (with every rank's fault
        words), root finalizes.  Hash group-bys (e.g. TPC-H Q3 by l_orderkey): every rank
        finalizes its groups, the rows are all-gathered to the root, which merges them
        with one more fused GROUP BY pipeline on its GPU (and applies ORDER BY / LIMIT)."""
        if getattr(pb, "root_only", False):  # no data collective: the root ran the whole pipeline
            self._root_only_checked(res)
            out = fetch(res, pb.result_names) if self.rank == self.root else None
        elif not hasattr(pb, "dist_order"):
            self._reduce_checked(res)
            out = fetch(res, pb.result_names) if self.rank == self.root else None
        else:
            out = self._merge_groups(res, pb)
        if self._trace is not None:
            self._trace_report("after fetch")
        return out

    def key_domain(self, table: str, col: str):
        """The key domain over ALL ranks' partitions (min / max all-reduced), so every rank
        declares the same group table."""
        lo, hi = self.tables[table].column_range(col)
        t = torch.tensor([-lo, hi], dtype=torch.int64, device=self.device)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        lo, hi = -int(t[0].item()), int(t[1].item())
        return (0, 1) if lo > hi else (lo, hi - lo + 1)

    def gather(self, res: Optional[hq.Result], pb: PlanBuilder) -> Optional[hq.Result]:
        """Complete result of a partitioned pipeline whose aggregation feeds a later build
        or root-side pipeline (e.g. TPC-H Q18's GROUP BY l_orderkey ... HAVING): hash
        group-bys are merged on the root (all-gather of the ranks' groups + one fused merge
        pipeline; an order split by the range partition is combined there), dense ones are
        summed with one all-reduce.  Returns the device result on the root, None elsewhere."""
        if getattr(pb, "root_only", False):
            return res
        if hasattr(pb, "dist_order"):
            merged = self._merge_device(res, pb)
            return merged[0] if merged is not None else None
        self._reduce_checked(res)
        return res if self.rank == self.root else None

    def _merge_groups(self, res: hq.Result, pb: PlanBuilder) -> Optional[QueryResult]:
        merged = self._merge_device(res, pb)
        if merged is None:
            return None
        out_res, mb, qual = merged
        out = fetch(out_res, mb.result_names)
        out.qualifying = qual  # rows that reached the sinks, over all ranks
        return out

    def _merge_device(self, res: hq.Result, pb: PlanBuilder):
        """All-gather the ranks' finalized groups; the root merges them with one fused
        GROUP BY pipeline (ORDER BY / LIMIT applied there).  Root: (result, plan, qualifying
        rows over all ranks); other ranks: None.  A rank whose local finalize fails (a
        pipeline fault) still takes part in the status all-reduce, then every rank raises."""
        P = pb.plan
        names = list(pb.result_names)
        # status = [qualifying rows, ranks that failed, fault words...], one SUM all-reduce
        st = torch.zeros(2 + hq.FAULT_WORDS, dtype=torch.int64, device=self.device)
        built, self._built = self._built, []
        self.ctx.gather_faults(built, [], st.data_ptr() + 16)  # the root's build faults
        err, tab, nrows = None, None, 0
        try:
            tab = res.as_table(names)  # finalized local groups (re-runs a full group table)
            nrows = tab.nrows
            st[0] = res.qualifying()
        except hq.HQError as e:
            err = e
            st[1] = 1
        dist.all_reduce(st)
        stl = st.tolist()
        if err is not None:
            raise err
        if stl[1]:
            raise RootError(hq.HQ_ERR_STATE, "pipeline failed on another rank")
        hq.raise_faults(stl[2:])
        qual = int(stl[0])
        ncol = len(names)
        n = torch.tensor([nrows], dtype=torch.int64, device=self.device)
        sizes = [torch.zeros_like(n) for _ in range(self.world)]
        dist.all_gather(sizes, n)
        sizes = [int(s.item()) for s in sizes]
        m = max(max(sizes), 1)
        # ONE all-gather of the packed [ncol, m] group rows
        pad = torch.zeros((ncol, m), dtype=torch.int64, device=self.device)
        for c in range(ncol):
            ptr, _ = tab.column_ptr(c)
            if nrows:
                pad[c, :nrows] = device_view(ptr, nrows * 8, torch.int64)
        bufs = [torch.empty_like(pad) for _ in range(self.world)]
        dist.all_gather(bufs, pad)
        if self.rank != self.root:
            return None
        merged = [torch.cat([b[c, :s] for b, s in zip(bufs, sizes)]).contiguous() for c in range(ncol)]
        mt = self.ctx.load_columns({nm: t for nm, t in zip(names, merged)})
        mb = PlanBuilder(mt)
        keys = [(names[i], P.key_min[i], P.key_card[i]) for i in range(P.nkeys)]
        fmap = {hq.AGG_SUM: "sum", hq.AGG_COUNT: "sum", hq.AGG_MIN: "min", hq.AGG_MAX: "max"}
        aggs = []
        for a in range(P.naggs):
            if P.agg_fn[a] not in fmap:
                raise NotImplementedError("distributed hash group-by merge: AVG needs SUM and COUNT partials")
            aggs.append((fmap[P.agg_fn[a]], names[P.nkeys + a]))
        order, limit = pb.dist_order
        mb.aggregate(keys=keys, aggs=aggs, order=[(names[c], bool(d)) for c, d in order], limit=limit,
                     group_capacity=max(1024, sum(sizes)), agg_names=names[P.nkeys:])
        mb.root_only = True
        return self.ctx.run(mb.plan, keep=mb.keep + [merged]), mb, qual
