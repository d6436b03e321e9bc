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

from typing import List, Optional, Sequence, Tuple

import torch
import torch.distributed as dist

from paper_conf_sigmod_funkebnmt18_b200 import hq
from paper_conf_sigmod_funkebnmt18_b200.engine import Engine, PlanBuilder, QueryResult, fetch


def partition(n: int, rank: int, world: int) -> Tuple[int, int]:
    """Row range of `rank` in a range partition of n rows over `world` ranks."""
    return n * rank // world, n * (rank + 1) // world


def _i64(u: int) -> int:
    """uint64 bit pattern as a signed int64 (torch.int64 transport)."""
    return u - (1 << 64) if u >= (1 << 63) else u


def broadcast_blob(meta: Optional[Sequence[int]], buf: Optional[torch.Tensor], nbytes_index: int,
                   root: int, device) -> Tuple[List[int], torch.Tensor]:
    """Broadcast a small int64 meta vector, then a byte buffer whose size is
    meta[nbytes_index].  Non-root ranks pass meta=None, buf=None."""
    rank = dist.get_rank()
    m = torch.zeros(16, dtype=torch.int64, device=device)
    if rank == root:
        m[: len(meta)] = torch.tensor(list(meta), dtype=torch.int64)
    dist.broadcast(m, src=root)
    meta_out = [int(x) for x in m.tolist()]
    nbytes = meta_out[nbytes_index]
    if rank != root:
        buf = torch.empty(nbytes, dtype=torch.uint8, device=device)
    dist.broadcast(buf, src=root)
    return meta_out, buf


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

    def _share_many(self, hs: Sequence[Optional[hq.Hash]]) -> List[hq.Hash]:
        """Broadcast several root-built tables: ONE broadcast of all their metadata (the
        root sends what it knows on the host; only the other ranks read it back), then one
        asynchronous broadcast per slot array, then the imports -- instead of a metadata
        broadcast and host read per table (each a stream sync)."""
        n = len(hs)
        meta = torch.zeros((max(n, 1), 16), dtype=torch.int64, device=self.device)
        views = []
        if self.rank == self.root:
            rows = []
            for h in hs:
                ptr, m = h.device_view()
                self._built.append(h)  # build faults are checked in finish()
                views.append(device_view(ptr, int(m.bytes)))
                rows.append([m.capacity, m.slot_words, m.npayload, m.nkeys, m.bytes, m.key_min, m.layout,
                             m.pay_min, m.pay_max, m.key_max] + [_i64(w) for w in m.pay_set] + [m.composite, 0])
            meta[:n] = torch.tensor(rows, dtype=torch.int64)
        dist.broadcast(meta, src=self.root)
        if self.rank == self.root:
            for v in views:
                dist.broadcast(v, src=self.root)
            return list(hs)
        rows = meta.cpu().tolist()
        out = []
        for r in rows[:n]:
            buf = torch.empty(int(r[4]), dtype=torch.uint8, device=self.device)
            dist.broadcast(buf, src=self.root)
            hm = hq.HashMeta()
            (hm.capacity, hm.slot_words, hm.npayload, hm.nkeys, hm.bytes, hm.key_min, hm.layout,
             hm.pay_min, hm.pay_max, hm.key_max) = r[:10]
            for k in range(4):
                hm.pay_set[k] = r[10 + k] & 0xFFFFFFFFFFFFFFFF
            hm.composite = r[14]
            out.append(self.ctx.import_hash(hm, buf.data_ptr(), keep=buf))
        return out

    def hash(self, table, key, payload=(), preds=(), expected_rows=0, key2=None) -> hq.Hash:
        h = super().hash(table, key, payload, preds, expected_rows, key2) if self.rank == self.root else None
        return self._share_many([h])[0]

    def hashes(self, specs) -> List[hq.Hash]:
        hs = super().hashes(specs) if self.rank == self.root else [None] * len(specs)
        return self._share_many(hs)

    def hash_from(self, res, names, key, payload=(), preds=()) -> hq.Hash:
        h = super().hash_from(res, names, key, payload, preds) if self.rank == self.root else None
        return self._share_many([h])[0]

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

    def finish(self, res: hq.Result, pb: PlanBuilder) -> Optional[QueryResult]:
        """Dense aggregates: one all-reduce of the partials, root finalizes.
        Hash group-bys (e.g. TPC-H Q3 by l_orderkey): every rank finalizes its
        groups, the rows are all-gathered to the root, which merges them with one
        more fused GROUP BY pipeline on its GPU (and applies ORDER BY / LIMIT)."""
        for h in self._built:  # root: raise duplicate-key / build faults (syncs)
            h.info()
        self._built.clear()
        if getattr(pb, "root_only", False):  # no collective: the root ran the whole pipeline
            return fetch(res, pb.result_names) if self.rank == self.root else None
        if not hasattr(pb, "dist_order"):
            ptr, nbytes = res.partials_view()
            t = device_view(ptr, nbytes, torch.int64)
            reduce_partials(t, self.root)
            if self.rank != self.root:
                return None
            return fetch(res, pb.result_names)
        return self._merge_groups(res, pb)

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
        ptr, nbytes = res.partials_view()
        reduce_partials(device_view(ptr, nbytes, torch.int64), self.root)
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
        rows over all ranks); other ranks: None."""
        P = pb.plan
        names = list(pb.result_names)
        tab = res.as_table(names)  # finalized local groups, device columns
        cols = []
        for c in range(len(names)):
            ptr, _ = tab.column_ptr(c)
            cols.append(device_view(ptr, max(tab.nrows, 1) * 8, torch.int64)[: tab.nrows])
        qual = torch.tensor([res.qualifying()], dtype=torch.int64, device=self.device)
        dist.all_reduce(qual)
        n = torch.tensor([tab.nrows], dtype=torch.int64, device=self.device)
        sizes = [torch.zeros_like(n) for _ in range(self.world)]
        dist.all_gather(sizes, n)
        sizes = [int(s.item()) for s in sizes]
        m = max(max(sizes), 1)
        merged = []
        for c in cols:
            pad = torch.zeros(m, dtype=torch.int64, device=self.device)
            pad[: c.numel()] = c
            bufs = [torch.empty_like(pad) for _ in range(self.world)]
            dist.all_gather(bufs, pad)
            merged.append(torch.cat([b[:s] for b, s in zip(bufs, sizes)]))
        if self.rank != self.root:
            return None
        mt = self.ctx.load_columns({nm: t.contiguous() for nm, t in zip(names, merged)})
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
        return self.ctx.run(mb.plan, keep=mb.keep + [merged]), mb, int(qual.item())
