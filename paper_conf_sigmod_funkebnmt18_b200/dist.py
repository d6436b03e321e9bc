"""Multi-GPU orchestration: one process per GPU.

* the fact table is range-partitioned: rank r owns rows [r*N/P, (r+1)*N/P);
  the generator is partition-invariant, so the union equals the P=1 input;
* dimension hash tables are built once on the root and broadcast as raw slot
  arrays (``hq_hash_device_view`` -> ``dist.broadcast`` over NCCL/NVLink ->
  ``hq_hash_import``); build-side pipelines (e.g. TPC-H Q3's orders side) run
  on the root only;
* each rank runs the fused pipeline over its range; dense partial aggregates
  ([count, agg...] per group, int64) are combined with ONE ``dist.reduce``
  (SUM) to the root, which finalizes (ORDER BY / LIMIT on GPU 0);
* replicated dimensions (``DistributedEngine(replicated=True)``, the bench's default):
  every rank holds the dimension tables and builds them itself -- no broadcast; only
  tables built over a result that exists on the root alone (after a gather) are sent;
* co-partitioned queries (``Query.copart``, TPC-H Q3): the order table and the line
  table are partitioned together by order (``hqgen.copartition``: rank r's lines are
  exactly the lines of its orders), every rank builds all of its tables locally (no
  broadcast: the orders table a rank probes holds only its own orders), its groups --
  keyed by the orderkey -- are disjoint from the other ranks', so ORDER BY / LIMIT run
  per rank and only the ranks' top-k rows are gathered and merged on the root.

The collectives here are backend-agnostic torch.distributed calls (NCCL on the
GPUs; the CPU tests drive the same functions with gloo and a test-only
stand-in for the device engine).  The paper itself is single-device; this is
new (north_star).
"""
from __future__ import annotations

import os
import sys
from typing import List, Optional, Sequence, Tuple

import numpy as np
import torch
import torch.distributed as dist

from . import hq
from .engine import Engine, PlanBuilder, QueryResult, fetch


def partition(n: int, rank: int, world: int) -> Tuple[int, int]:
    """Row range of `rank` in a range partition of n rows over `world` ranks."""
    return n * rank // world, n * (rank + 1) // world


def run_query(E: Engine, q) -> Optional[QueryResult]:
    """One query through an Engine or DistributedEngine: q.run + finish, with the
    co-partitioned abort protocol (a rank that raises joins the status collective)."""
    try:
        res, pb = q.run(E)
    except hq.HQError as e:
        if isinstance(E, DistributedEngine) and E.copartitioned:
            E.abort(e)
        raise
    return E.finish(res, pb)


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


# The step's collectives go straight to the default process group (its broadcast /
# allreduce methods): the torch.distributed wrappers (argument checks, the c10d logger)
# cost ~50-100 us of host time per call, which a step's critical path pays (the table
# broadcast sits between the builds and the pipeline launch).  Same semantics as the
# synchronous dist.* calls: work.wait() makes the current stream wait for the collective.
def _pg():
    return dist.distributed_c10d._get_default_group()


def _broadcast(t: torch.Tensor, src: int) -> None:
    opts = dist.BroadcastOptions()
    opts.rootRank = src
    opts.rootTensor = 0
    _pg().broadcast([t], opts).wait()


def _all_reduce(t: torch.Tensor, op=dist.ReduceOp.SUM) -> None:
    opts = dist.AllreduceOptions()
    opts.reduceOp = op
    _pg().allreduce([t], opts).wait()


def _align(x: int, a: int = 256) -> int:
    return (x + a - 1) // a * a


def broadcast_tables(rows: Optional[List[List[int]]], pack, n: int, root: int, device,
                     err: Optional[BaseException] = None, state: Optional[dict] = None
                     ) -> Tuple[List[List[int]], List[torch.Tensor]]:
    """Broadcast n root-built tables, normally with ONE collective: a byte buffer
    [(n+1) x 16 int64 metadata (row n = the root's status) | every table's buffer at a
    256-B aligned offset].  The other ranks size their receive buffer from ``state``
    (the largest message so far, the same on every rank); when the root's message is
    larger, the first broadcast carries only the metadata with the new size in row n,
    and a second one the whole message.  Root: rows and ``pack`` given -- a list of
    tensors, or a callable(dev_ptr, offsets) that copies the tables into the buffer
    (hq_hash_pack); other ranks: None (they get views into the received buffer).  A
    root-side error is broadcast before the root re-raises it, so the other ranks raise
    RootError instead of blocking in the next collective."""
    rank = dist.get_rank()
    st = state if state is not None else {}
    hdr = _align((n + 1) * META_COLS * 8)
    first = max(int(st.get("cap", 0)), hdr)
    if rank == root:
        offs, tot = _offsets(rows) if (err is None and n) else ([], 0)
        need = hdr + tot
        grow = need > first
        meta = np.zeros((n + 1, META_COLS), dtype=np.int64)
        if err is not None:
            meta[n, 0] = getattr(err, "code", hq.HQ_ERR_STATE) or hq.HQ_ERR_STATE
        elif n:
            meta[:n] = np.asarray(rows, dtype=np.int64)
            meta[n, 1] = need if grow else 0
        buf = torch.empty(max(first, need), dtype=torch.uint8, device=device)
        host = torch.from_numpy(meta.view(np.uint8).ravel())
        if buf.is_cuda:  # pinned staging, reused (steps synchronise before the next call)
            ph = st.get("pinned")
            if ph is None or ph.numel() < host.numel():
                ph = st["pinned"] = torch.empty(max(host.numel(), 4096), dtype=torch.uint8, pin_memory=True)
            ph[:host.numel()].copy_(host)
            host = ph[:host.numel()]
        buf[:host.numel()].copy_(host, non_blocking=True)

        def fill():
            base = hdr
            if callable(pack):
                pack(buf.data_ptr() + base, offs)
            else:
                for o, b in zip(offs, pack):
                    buf[base + o:base + o + b.numel()].copy_(b.reshape(-1).view(torch.uint8))
        if err is None and n and not grow:
            fill()
        _broadcast(buf[:first], root)
        if err is not None:
            raise err
        if grow:
            fill()
            _broadcast(buf[:need], root)
            st["cap"] = need
        return rows, ([] if not n else list(pack) if not callable(pack) else [])
    buf = torch.empty(first, dtype=torch.uint8, device=device)
    _broadcast(buf, root)
    m = buf[:(n + 1) * META_COLS * 8].view(torch.int64).reshape(n + 1, META_COLS).cpu().tolist()
    if m[n][0] != 0:
        raise RootError(int(m[n][0]), "hash build failed on the root rank")
    rows = m[:n]
    if n == 0:
        return rows, []
    need = int(m[n][1])
    if need:
        buf = torch.empty(need, dtype=torch.uint8, device=device)
        _broadcast(buf, root)
        st["cap"] = need
    offs, _ = _offsets(rows)
    return rows, [buf[hdr + o:hdr + o + int(r[4])] for o, r in zip(offs, rows)]


def reduce_partials(t: torch.Tensor, root: int) -> None:
    """Exact integer SUM of the ranks' partial aggregates (one all-reduce: NCCL
    over NVLink on the GPUs; gloo in the CPU tests).  Only the root finalizes."""
    _all_reduce(t)


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

    def __init__(self, ctx: hq.Context, tables, root: int = 0, copartitioned: bool = False, replicated: bool = False,
                 **kw):
        super().__init__(ctx, tables, **kw)
        self.rank = dist.get_rank()
        self.world = dist.get_world_size()
        self.root = root
        self.device = torch.device("cuda", ctx.device)
        self._built: List[hq.Hash] = []
        self._bcast: dict = {}  # broadcast_tables state (receive size), identical on every rank
        # copartitioned: the tables are this rank's co-partition (hqgen.copartition) plus
        # full copies of the small dimensions; every rank builds and runs locally
        self.copartitioned = copartitioned
        # replicated: every rank holds the full dimension tables (the fact table stays range-
        # partitioned) and runs the build side itself -- builds over base tables and the
        # unpartitioned pipelines over them -- so no table is broadcast; only builds over a
        # result that exists on the root alone (after a gather) still are
        self.replicated = replicated
        self._local_results: set = set()  # ids of results every rank computed itself
        self.builds_here = copartitioned or replicated or self.rank == root
        # HQ_DIST_FAULT_TRACE=1 (debug): re-read every root build's fault word after the
        # final fetch and report the ones that changed since the build
        self._trace: Optional[List[Tuple[str, hq.Hash, List[int]]]] = (
            [] if os.environ.get("HQ_DIST_FAULT_TRACE") == "1" else None)

    def _share_many(self, hs: Optional[Sequence[hq.Hash]], n: int, err: Optional[BaseException] = None) -> List[hq.Hash]:
        """Broadcast n root-built tables (broadcast_tables: metadata and every table in one
        buffer, normally one collective; the root packs them with hq_hash_pack, no host
        read on the root) and import them on the other ranks.  Build faults are not read
        here (that would sync per table): the root's fault words travel with the
        pipeline's reduce (_reduce_checked)."""
        if self.rank == self.root:
            rows = []
            if err is None:
                for h in hs:
                    _, m = h.device_view()
                    self._built.append(h)
                    if self._trace is not None:
                        self._trace.append((f"build#{len(self._trace)} rows={m.nkeys} cap={m.capacity}", h,
                                            self._faults_of(h)))
                    rows.append(meta_row(m))
            hl = list(hs) if hs is not None else []
            broadcast_tables(rows, lambda ptr, offs: self.ctx.pack_hashes(hl, offs, ptr), n, self.root, self.device,
                             err, self._bcast)
            return hl
        rows, bufs = broadcast_tables(None, None, n, self.root, self.device, state=self._bcast)
        return [self.ctx.import_hash(meta_from_row(r), b.data_ptr(), keep=b) for r, b in zip(rows, bufs)]  # views keep the buffer

    def _root_build(self, fn, n: int, local: bool = False):
        if self.copartitioned or local:  # built on every rank from data it holds: nothing to share
            hs = fn()
            self._built.extend(hs)
            return hs
        hs, err = None, None
        if self.rank == self.root:
            try:
                hs = fn()
            except hq.HQError as e:
                err = e
        return self._share_many(hs, n, err)

    def hash(self, table, key, payload=(), preds=(), expected_rows=0, key2=None) -> hq.Hash:
        return self._root_build(lambda: [super(DistributedEngine, self).hash(table, key, payload, preds,
                                                                             expected_rows, key2)], 1,
                                self.replicated)[0]

    def hashes(self, specs) -> List[hq.Hash]:
        return self._root_build(lambda: super(DistributedEngine, self).hashes(specs), len(specs), self.replicated)

    def hash_from(self, res, names, key, payload=(), preds=()) -> hq.Hash:
        local = self.replicated and res is not None and id(res) in self._local_results
        return self._root_build(lambda: [super(DistributedEngine, self).hash_from(res, names, key, payload,
                                                                                  preds)], 1, local)[0]

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
        if self.copartitioned:
            if not partitioned:  # a build-side pipeline over this rank's co-partition
                return super().run(pb, partitioned)
            P = pb.plan
            if not self._hash_grouped(P):
                raise NotImplementedError("co-partitioned execution: the final pipeline must group by the "
                                          "co-partitioning key (hash group-by)")
            # groups are disjoint across ranks: ORDER BY / LIMIT stay in the local plan,
            # the root merges the ranks' top rows
            pb.dist_order = ([(P.order_col[i], P.order_desc[i]) for i in range(P.norder)], P.limit)
            pb.copart_local_order = True
            return super().run(pb, partitioned)
        if not partitioned and self.replicated and any(pb.fact is t for t in self.tables.values()):
            # a build-side pipeline over (replicated) base tables: every rank runs it
            res = super().run(pb, partitioned)
            pb.replicated_local = True
            self._local_results.add(id(res))
            pb.keep.append(res)  # (keeps the id valid while the plan lives)
            return res
        if not partitioned:
            pb.root_only = True  # a build-side or post-merge pipeline: the root's result is complete
            if self.rank != self.root:
                return None
            return super().run(pb, partitioned)
        P = pb.plan
        if partitioned and P.sink == hq.SINK_MATERIALISE:
            pb.dist_rows = True  # each rank materialises its rows; finish() gathers them to the root
        if partitioned and self._hash_grouped(P):
            # ranks keep all their groups; ORDER BY / LIMIT run after the root's merge
            pb.dist_order = ([(P.order_col[i], P.order_desc[i]) for i in range(P.norder)], P.limit)
            P.norder, P.limit = 0, 0
        return super().run(pb, partitioned)

    def prepare(self, query, **kw) -> "PreparedDistQuery":
        """A prepared distributed step (replicated dimensions, a dense final aggregation):
        two CUDA graphs around the collective -- the builds, the pipeline and the packing
        of [partials | fault words] into a persistent buffer; the all-reduce on the device
        between them; the partials' copy-back and the finalize.  Raises HQError(HQ_ERR_STATE)
        or NotImplementedError for steps it cannot hold (the caller runs them eagerly)."""
        return PreparedDistQuery(self, query, **kw)

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

    def _reduce_checked(self, res: hq.Result, defer: bool = False) -> Optional[torch.Tensor]:
        """ONE all-reduce of [dense partials | fault words]: the partials are summed
        (exact int64), and the fault words -- the root's build faults and every rank's
        pipeline faults, gathered on the device (hq_gather_faults) -- are summed too, so
        every rank sees every rank's faults and raises, or none does.  One host read of
        the 32 fault words at the end; no per-table synchronisation.  defer: the words are
        copied to pinned host memory asynchronously and returned; the caller raises them
        after its next synchronisation (the root's fetch), saving a host round trip."""
        ptr, nbytes = res.partials_view()
        n = nbytes // 8
        red = torch.empty(n + hq.FAULT_WORDS, dtype=torch.int64, device=self.device)
        res.to_partials(red.data_ptr(), nbytes)
        built, self._built = self._built, []
        self.ctx.gather_faults(built, [res], red.data_ptr() + n * 8)
        reduce_partials(red, self.root)
        res.from_partials(red.data_ptr(), nbytes)
        self._checked_built = built
        if not defer:
            self._raise(red[n:].tolist(), built)
            return None
        if getattr(self, "_fault_host", None) is None:
            self._fault_host = torch.empty(hq.FAULT_WORDS, dtype=torch.int64, pin_memory=True)
        self._fault_host.copy_(red[n:], non_blocking=True)
        self._fault_event = torch.cuda.Event()
        self._fault_event.record(torch.cuda.current_stream(self.device))
        return self._fault_host

    def _raise_deferred(self, words: torch.Tensor, built: Sequence[hq.Hash] = ()) -> None:
        self._fault_event.synchronize()  # (already complete after the root's fetch)
        self._raise(words.tolist(), built)

    @staticmethod
    def _raise(words: Sequence[int], built: Sequence[hq.Hash]) -> None:
        """hq.raise_faults; on stale build statistics, the tables this rank built are
        checked first (hq_hash_info), which drops their cached statistics so that the
        next run counts afresh instead of failing again."""
        try:
            hq.raise_faults(words)
        except hq.HQError as e:
            if e.code == hq.HQ_ERR_STATE:
                for h in built:
                    try:
                        h.info()
                    except hq.HQError:
                        pass
            raise

    def _root_only_checked(self, res: Optional[hq.Result]) -> None:
        """A root-only final pipeline: the root's build and pipeline faults are shared
        with one small all-reduce, so that all ranks raise together."""
        st = torch.zeros(hq.FAULT_WORDS, dtype=torch.int64, device=self.device)
        built, self._built = self._built, []
        if self.rank == self.root:
            self.ctx.gather_faults(built, [res] if res is not None else [], st.data_ptr())
        _all_reduce(st)
        self._raise(st.tolist(), built)

    def finish(self, res: hq.Result, pb: PlanBuilder) -> Optional[QueryResult]:
        """Dense aggregates: one all-reduce of the partials (with every rank's fault
        words), root finalizes.  Hash group-bys (e.g. TPC-H Q3 by l_orderkey): every rank
        finalizes its groups, the rows are all-gathered to the root, which merges them
        with one more fused GROUP BY pipeline on its GPU (and applies ORDER BY / LIMIT)."""
        if getattr(pb, "replicated_local", False):  # every rank computed the whole result
            if self.rank != self.root:
                res.finalize()  # (the same faults as the root's: every rank raises, or none)
            self._built = []
            out = fetch(res, pb.result_names) if self.rank == self.root else None
        elif getattr(pb, "root_only", False):  # no data collective: the root ran the whole pipeline
            self._root_only_checked(res)
            out = fetch(res, pb.result_names) if self.rank == self.root else None
        elif getattr(pb, "dist_rows", False):
            out = self._gather_rows(res, pb)
        elif not hasattr(pb, "dist_order"):
            words = self._reduce_checked(res, defer=True)
            try:
                out = fetch(res, pb.result_names) if self.rank == self.root else None
            finally:  # every rank raises the summed faults (before a fetch error)
                self._raise_deferred(words, self._checked_built)
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
        _all_reduce(t, dist.ReduceOp.MAX)
        lo, hi = -int(t[0].item()), int(t[1].item())
        return (0, 1) if lo > hi else (lo, hi - lo + 1)

    def abort(self, err: BaseException) -> None:
        """A co-partitioned rank whose local builds or pipeline raised on the host: join
        the first collective of finish() (the status all-reduce) with the failure flag
        set, so the other ranks raise RootError instead of waiting; then re-raise."""
        st = torch.zeros(2 + hq.FAULT_WORDS, dtype=torch.int64, device=self.device)
        st[1] = 1
        self._built = []
        _all_reduce(st)
        raise err

    def gather(self, res: Optional[hq.Result], pb: PlanBuilder) -> Optional[hq.Result]:
        """Complete result of a partitioned pipeline whose aggregation feeds a later build
        or root-side pipeline (e.g. TPC-H Q18's GROUP BY l_orderkey ... HAVING): hash
        group-bys are merged on the root (all-gather of the ranks' groups + one fused merge
        pipeline; an order split by the range partition is combined there), dense ones are
        summed with one all-reduce.  Returns the device result on the root, None elsewhere."""
        if getattr(pb, "root_only", False) or getattr(pb, "replicated_local", False):
            return res
        if self.copartitioned:
            raise NotImplementedError("co-partitioned execution: intermediate gathers are not supported")
        if hasattr(pb, "dist_order"):
            merged = self._merge_device(res, pb)
            return merged[0] if merged is not None else None
        self._reduce_checked(res)
        return res if self.rank == self.root else None

    def _gather_rows(self, res: hq.Result, pb: PlanBuilder) -> Optional[QueryResult]:
        """A partitioned materialising pipeline (SURVEY §8(e) "materialise sinks"): one
        status all-reduce (row counts, failures, fault words), one all-gather of each
        rank's rows packed as int64 [ncols, m], the root concatenates them (each rank's
        rows one segment; the segments in rank order) and casts back to the column types."""
        names = list(pb.result_names)
        st = torch.zeros(2 + hq.FAULT_WORDS, dtype=torch.int64, device=self.device)
        built, self._built = self._built, []
        self.ctx.gather_faults(built, [], st.data_ptr() + 16)
        err, tab, nrows = None, None, 0
        try:
            tab = res.as_table(names)
            nrows = tab.nrows
            st[0] = res.qualifying()
        except hq.HQError as e:
            err = e
            st[1] = 1
        _all_reduce(st)
        stl = st.tolist()
        if err is not None:
            raise err
        if stl[1]:
            raise RootError(hq.HQ_ERR_STATE, "pipeline failed on another rank")
        self._raise(stl[2:], built)
        ncol = len(names)
        n = torch.tensor([nrows], dtype=torch.int64, device=self.device)
        sizes = [torch.zeros_like(n) for _ in range(self.world)]
        dist.all_gather(sizes, n)
        sizes = [int(x.item()) for x in sizes]
        m = max(max(sizes), 1)
        pad = torch.zeros((ncol, m), dtype=torch.int64, device=self.device)
        types = []
        for c in range(ncol):
            ptr, t = tab.column_ptr(c)
            dt = {hq.HQ_I8: torch.int8, hq.HQ_I32: torch.int32, hq.HQ_I64: torch.int64}[t]
            types.append(dt)
            if nrows:
                w = torch.empty((), dtype=dt).element_size()
                v = device_view(ptr, nrows * w, torch.uint8).view(dt)
                pad[c, :nrows] = v.to(torch.int64)
        bufs = [torch.empty_like(pad) for _ in range(self.world)]
        dist.all_gather(bufs, pad)
        if self.rank != self.root:
            return None
        cols = {nm: torch.cat([b[c, :sz] for b, sz in zip(bufs, sizes)]).to(types[c]).cpu().numpy()
                for c, nm in enumerate(names)}
        return QueryResult(cols, int(stl[0]))

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
        err, tab, nrows, cols = None, None, 0, None
        local_top = getattr(pb, "copart_local_order", False)
        try:
            if local_top:  # disjoint groups: this rank's ORDER BY / LIMIT rows are final candidates
                top = fetch(res, names)
                if any(top.columns[nm].dtype.kind == "f" for nm in names):
                    raise hq.HQError(hq.HQ_ERR_UNSUPPORTED, "co-partitioned merge: fp64 (AVG) result column")
                nrows = top.nrows
                cols = torch.from_numpy(np.stack([np.asarray(top.columns[nm], dtype=np.int64) for nm in names])
                                        if nrows else np.zeros((len(names), 0), np.int64))
                st[0] = top.qualifying
            else:
                tab = res.as_table(names)  # finalized local groups (re-runs a full group table)
                nrows = tab.nrows
                st[0] = res.qualifying()
        except hq.HQError as e:
            err = e
            st[1] = 1
        _all_reduce(st)
        stl = st.tolist()
        if err is not None:
            raise err
        if stl[1]:
            raise RootError(hq.HQ_ERR_STATE, "pipeline failed on another rank")
        self._raise(stl[2:], built)
        qual = int(stl[0])
        ncol = len(names)
        n = torch.tensor([nrows], dtype=torch.int64, device=self.device)
        sizes = [torch.zeros_like(n) for _ in range(self.world)]
        dist.all_gather(sizes, n)
        sizes = [int(s.item()) for s in sizes]
        m = max(max(sizes), 1)
        # ONE all-gather of the packed [ncol, m] group rows
        pad = torch.zeros((ncol, m), dtype=torch.int64, device=self.device)
        if cols is not None:
            pad[:, :nrows] = cols.to(self.device)
        else:
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


class PreparedDistQuery:
    """DistributedEngine.prepare: graph A (builds + fused pipeline + partials and fault
    words packed into a persistent device buffer), the all-reduce of that buffer over the
    process group, graph B (partials copied back, finalize).  Graph A launches
    asynchronously, so the collective's host call overlaps the pipeline.  Every launch
    re-executes all device work; the fault words are read after B's synchronisation and
    raised on every rank together."""

    def __init__(self, E: DistributedEngine, query, **kw):
        if not E.replicated or E.copartitioned:
            raise NotImplementedError("prepared distributed steps need replicated dimensions")
        self.E, self.query = E, query
        run_query(E, query)  # eager: kernels compiled, build statistics and result views cached
        ctx = E.ctx
        E._built = []
        ctx.capture_begin()
        try:
            res, pb = query.run(E, **kw)
            if res is None or getattr(pb, "dist_rows", False) or hasattr(pb, "dist_order") or \
                    getattr(pb, "root_only", False) or getattr(pb, "replicated_local", False):
                raise NotImplementedError("prepared distributed steps: a dense final aggregation only")
            ptr, nbytes = res.partials_view()
            self.n = nbytes // 8
            self.red = torch.zeros(self.n + hq.FAULT_WORDS, dtype=torch.int64, device=E.device)
            res.to_partials(self.red.data_ptr(), nbytes)
            built, E._built = E._built, []
            ctx.gather_faults(built, [res], self.red.data_ptr() + self.n * 8)
        except BaseException:
            ctx.capture_abort()
            E._built = []
            raise
        self.graph_a = ctx.capture_end()
        self.built = built
        ctx.capture_begin()
        try:
            res.from_partials(self.red.data_ptr(), nbytes)
            res.finalize()
        except BaseException:
            ctx.capture_abort()
            self.graph_a.free()
            raise
        self.graph_b = ctx.capture_end()
        self.res, self.pb = res, pb
        self.words = torch.empty(hq.FAULT_WORDS, dtype=torch.int64, pin_memory=True)

    def execute(self) -> Optional[QueryResult]:
        E = self.E
        self.graph_a.launch()  # asynchronous
        _all_reduce(self.red)  # the device-side collective, ordered after graph A
        self.words.copy_(self.red[self.n:], non_blocking=True)
        self.graph_b.launch()  # synchronises (the finalized rows are decoded on the host)
        E._raise(self.words.tolist(), self.built)
        return fetch(self.res, self.pb.result_names) if E.rank == E.root else None

    def close(self) -> None:
        self.graph_a.free()
        self.graph_b.free()
