"""ctypes binding of libhq (include/hq.h) -- argument marshalling only.

Every step of a query runs in libhq's CUDA kernels; this module mirrors the C
structs, owns handles and maps status codes to exceptions.  There is no CPU
fallback: if ``libhq.so`` is missing or no CUDA device is present, the calls
raise (``HQ_ERR_NO_DEVICE``).  PyTorch is used for device memory (optional
caching-allocator hooks) and streams only.
"""
from __future__ import annotations

import ctypes
import os
from typing import Dict, List, Optional, Sequence

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
SO_PATH = os.environ.get("HQ_LIB_PATH") or os.path.join(_PKG, "libhq.so")  # override: debugging only

# ---- constants (mirror hq.h) ----------------------------------------------
HQ_OK, HQ_ERR_ARG, HQ_ERR_CUDA, HQ_ERR_OOM, HQ_ERR_DUP_KEY = 0, -1, -2, -3, -4
HQ_ERR_UNSUPPORTED, HQ_ERR_OVERFLOW, HQ_ERR_STATE, HQ_ERR_NO_DEVICE = -5, -6, -7, -8
HQ_I8, HQ_I32, HQ_I64, HQ_F64 = 1, 3, 4, 5
MAX_COLS, MAX_OPS, MAX_PAYLOAD, MAX_KEYS, MAX_AGGS = 16, 16, 3, 4, 8
MAX_OUT, MAX_TMP, MAX_INSN, MAX_PREDS, MAX_ORDER = 8, 8, 16, 8, 4
HQ_HOST_COPY, HQ_DEVICE_BORROW, HQ_HOST_STREAM = 1, 2, 3
STREAM_BLOCK_ROWS = 1 << 24
EQ, NE, LT, LE, GT, GE, BETWEEN, IN_BITMAP = 1, 2, 3, 4, 5, 6, 7, 8
OP_FILTER, OP_PROBE, OP_COMPUTE = 1, 2, 3
PROBE_INNER, PROBE_SEMI, PROBE_ANTI, PROBE_OUTER = 0, 1, 2, 3
I_LOAD, I_ADD, I_SUB, I_RSUB, I_MUL, I_DIV, I_MOD = 1, 2, 3, 4, 5, 6, 7
I_AND_EQ, I_AND_NE, I_AND_LT, I_AND_LE, I_AND_GT, I_AND_GE, I_AND_IN, I_OR = 8, 9, 10, 11, 12, 13, 14, 15
AGG_SUM, AGG_COUNT, AGG_MIN, AGG_MAX, AGG_AVG = 1, 2, 3, 4, 5
SINK_AGG, SINK_MATERIALISE = 1, 2
RES_LRGP, RES_ATOMIC, RES_WE = 0, 1, 2
EXEC_FUSED, EXEC_OAAT, EXEC_FUSED_INTERP, EXEC_MULTIPASS = 0, 1, 2, 3
HT_LINEAR, HT_DIRECT = 0, 1  # hq_hash_meta.layout


def TMP(k: int) -> int:
    return 0x100 + k


DTYPE_TO_HQ = {np.dtype(np.int8): HQ_I8, np.dtype(np.int32): HQ_I32, np.dtype(np.int64): HQ_I64}
HQ_TO_DTYPE = {HQ_I8: np.int8, HQ_I32: np.int32, HQ_I64: np.int64, HQ_F64: np.float64}
HQ_WIDTH = {HQ_I8: 1, HQ_I32: 4, HQ_I64: 8, HQ_F64: 8}


# ---- struct mirrors ---------------------------------------------------------
class Column(ctypes.Structure):
    _fields_ = [("name", ctypes.c_char_p), ("type", ctypes.c_int32), ("reserved", ctypes.c_int32),
                ("data", ctypes.c_void_p)]


class Pred(ctypes.Structure):
    _fields_ = [("reg", ctypes.c_int32), ("cmp", ctypes.c_int32), ("lo", ctypes.c_int64),
                ("hi", ctypes.c_int64), ("bitmap", ctypes.c_uint64 * 4)]


class BuildDesc(ctypes.Structure):
    _fields_ = [("src", ctypes.c_void_p), ("npreds", ctypes.c_int32), ("preds", Pred * MAX_PREDS),
                ("key_col", ctypes.c_int32), ("npayload", ctypes.c_int32),
                ("payload_cols", ctypes.c_int32 * MAX_PAYLOAD), ("expected_rows", ctypes.c_int64),
                ("composite", ctypes.c_int32)]


class HashMeta(ctypes.Structure):
    _fields_ = [("capacity", ctypes.c_int64), ("slot_words", ctypes.c_int32), ("npayload", ctypes.c_int32),
                ("nkeys", ctypes.c_int64), ("bytes", ctypes.c_int64), ("key_min", ctypes.c_int64),
                ("layout", ctypes.c_int32), ("pay_min", ctypes.c_int32), ("pay_max", ctypes.c_int32),
                ("key_max", ctypes.c_int32), ("pay_set", ctypes.c_uint64 * 4), ("composite", ctypes.c_int32),
                ("compact_kind", ctypes.c_int32)]


class Insn(ctypes.Structure):
    _fields_ = [("opc", ctypes.c_int32), ("reg", ctypes.c_int32), ("imm", ctypes.c_int64)]


class Op(ctypes.Structure):
    _fields_ = [("kind", ctypes.c_int32), ("filter", Pred), ("ht", ctypes.c_void_p),
                ("key_reg", ctypes.c_int32), ("mode", ctypes.c_int32), ("npayload", ctypes.c_int32),
                ("payload_dst", ctypes.c_int32 * MAX_PAYLOAD), ("dst", ctypes.c_int32),
                ("ninsn", ctypes.c_int32), ("code", Insn * MAX_INSN), ("key2_reg", ctypes.c_int32)]


class Plan(ctypes.Structure):
    _fields_ = [("fact", ctypes.c_void_p), ("row_begin", ctypes.c_int64), ("row_end", ctypes.c_int64),
                ("nops", ctypes.c_int32), ("ops", Op * MAX_OPS), ("sink", ctypes.c_int32),
                ("resolution", ctypes.c_int32), ("exec", ctypes.c_int32), ("ntmp_types", ctypes.c_int32),
                ("nkeys", ctypes.c_int32), ("key_reg", ctypes.c_int32 * MAX_KEYS),
                ("key_min", ctypes.c_int64 * MAX_KEYS), ("key_card", ctypes.c_int64 * MAX_KEYS),
                ("naggs", ctypes.c_int32), ("agg_fn", ctypes.c_int32 * MAX_AGGS),
                ("agg_reg", ctypes.c_int32 * MAX_AGGS), ("agg_scale", ctypes.c_int32 * MAX_AGGS),
                ("group_capacity", ctypes.c_int64), ("nout", ctypes.c_int32),
                ("out_reg", ctypes.c_int32 * MAX_OUT), ("out_type", ctypes.c_int32 * MAX_OUT),
                ("capacity", ctypes.c_int64), ("norder", ctypes.c_int32),
                ("order_col", ctypes.c_int32 * MAX_ORDER), ("order_desc", ctypes.c_int32 * MAX_ORDER),
                ("limit", ctypes.c_int64)]


class ResultInfo(ctypes.Structure):
    _fields_ = [("nrows", ctypes.c_int64), ("qualifying_rows", ctypes.c_int64), ("ncols", ctypes.c_int32),
                ("types", ctypes.c_int32 * (MAX_KEYS + MAX_AGGS)), ("segment_rows", ctypes.c_int32)]


ALLOC_FN = ctypes.CFUNCTYPE(ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p, ctypes.c_void_p)
FREE_FN = ctypes.CFUNCTYPE(None, ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p, ctypes.c_void_p)


class Allocator(ctypes.Structure):
    _fields_ = [("alloc", ALLOC_FN), ("free", FREE_FN), ("user", ctypes.c_void_p)]


STRUCTS = {"hq_column": Column, "hq_pred": Pred, "hq_build_desc": BuildDesc, "hq_hash_meta": HashMeta,
           "hq_insn": Insn, "hq_op": Op, "hq_plan": Plan, "hq_result_info": ResultInfo,
           "hq_allocator": Allocator}

# every symbol include/hq.h declares
EXPORTS = ["hq_ctx_create", "hq_ctx_destroy", "hq_ctx_set_stream", "hq_ctx_sync", "hq_last_error",
           "hq_abi_version", "hq_sizeof", "hq_ctx_enable_timing", "hq_ctx_kernel_times", "hq_ctx_launches",
           "hq_load_columns", "hq_column_range",
           "hq_table_info", "hq_table_column", "hq_free_table", "hq_build_hash", "hq_build_hashes", "hq_hash_info",
           "hq_hash_device_view", "hq_hash_import", "hq_free_hash", "hq_run_pipeline", "hq_run_pipeline_streamed",
           "hq_finalize",
           "hq_result_info_get", "hq_fetch_result", "hq_result_as_table", "hq_result_partials_view",
           "hq_result_from_partials", "hq_result_to_partials", "hq_hash_pack", "hq_gather_faults", "hq_raise_faults", "hq_free_result",
           "hq_ctx_capture_begin", "hq_ctx_capture_end", "hq_ctx_capture_abort", "hq_graph_launch", "hq_graph_destroy"]
FAULT_WORDS = 32


class HQError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"libhq error {code}: {msg}")
        self.code = code


_lib = None


def lib():
    """Load libhq.so (never builds, never falls back)."""
    global _lib
    if _lib is None:
        if not os.path.exists(SO_PATH):
            raise RuntimeError(f"{SO_PATH} is missing: run __graft_entry__.build() (no CPU fallback)")
        L = ctypes.CDLL(SO_PATH)
        P, vp, i32, i64 = ctypes.POINTER, ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64
        sig = {
            "hq_ctx_create": [i32, vp, P(Allocator), P(vp)],
            "hq_ctx_destroy": [vp], "hq_ctx_set_stream": [vp, vp], "hq_ctx_sync": [vp],
            "hq_ctx_enable_timing": [vp, i32],
            "hq_ctx_kernel_times": [vp, P(ctypes.c_float), i32, P(i32)],
            "hq_ctx_launches": [vp, P(i64)],
            "hq_load_columns": [vp, P(Column), i32, i64, i32, P(vp)],
            "hq_table_info": [vp, P(i64), P(i32)], "hq_table_column": [vp, i32, P(vp), P(i32)],
            "hq_free_table": [vp], "hq_build_hash": [vp, P(BuildDesc), P(vp)],
            "hq_build_hashes": [vp, i32, P(BuildDesc), P(vp)],
            "hq_hash_info": [vp, vp, P(HashMeta)], "hq_hash_device_view": [vp, P(vp), P(HashMeta)],
            "hq_hash_import": [vp, P(HashMeta), vp, P(vp)], "hq_free_hash": [vp],
            "hq_run_pipeline": [vp, P(Plan), P(vp)], "hq_finalize": [vp, vp],
            "hq_run_pipeline_streamed": [vp, P(Plan), i64, P(vp)],
            "hq_column_range": [vp, vp, i32, P(i64), P(i64)],
            "hq_result_info_get": [vp, vp, P(ResultInfo)],
            "hq_fetch_result": [vp, vp, P(vp), i64, P(i64)],
            "hq_result_as_table": [vp, vp, P(vp)],
            "hq_result_partials_view": [vp, P(vp), P(ctypes.c_size_t)], "hq_free_result": [vp],
            "hq_result_from_partials": [vp, vp, vp, ctypes.c_size_t],
            "hq_result_to_partials": [vp, vp, vp, ctypes.c_size_t],
            "hq_hash_pack": [vp, P(vp), i32, P(i64), vp],
            "hq_gather_faults": [vp, P(vp), i32, P(vp), i32, vp],
            "hq_raise_faults": [P(i64)],
            "hq_ctx_capture_begin": [vp], "hq_ctx_capture_end": [vp, P(vp)], "hq_ctx_capture_abort": [vp],
            "hq_graph_launch": [vp, vp], "hq_graph_destroy": [vp],
        }
        for name, args in sig.items():
            f = getattr(L, name, None)
            if f is None:  # an older library (HQ_LIB_PATH): the call is unavailable
                continue
            f.argtypes = args
            f.restype = ctypes.c_int32
        L.hq_last_error.restype = ctypes.c_char_p
        L.hq_last_error.argtypes = []
        L.hq_abi_version.restype = ctypes.c_int32
        L.hq_sizeof.restype = ctypes.c_size_t
        L.hq_sizeof.argtypes = [ctypes.c_char_p]
        _lib = L
    return _lib


def check(status: int) -> None:
    if status != HQ_OK:
        raise HQError(status, lib().hq_last_error().decode(errors="replace"))


# ---- handles ----------------------------------------------------------------
class Context:
    """One libhq context per device/stream.  stream: a torch.cuda.Stream, a raw
    cudaStream_t int, or None (torch's current stream if torch is importable)."""

    def __init__(self, device: int = 0, stream=None, torch_allocator: bool = False):
        self.device = device
        raw = self._raw_stream(stream, device)
        self._alloc_keep = None
        alloc_p = None
        if torch_allocator:
            import torch

            def _a(n, s, u):
                return torch.cuda.caching_allocator_alloc(int(n), device, s)

            def _f(p, n, s, u):
                torch.cuda.caching_allocator_delete(p)

            self._alloc_keep = Allocator(ALLOC_FN(_a), FREE_FN(_f), None)
            alloc_p = ctypes.byref(self._alloc_keep)
        h = ctypes.c_void_p()
        check(lib().hq_ctx_create(device, raw, alloc_p, ctypes.byref(h)))
        self.h = h

    @staticmethod
    def _raw_stream(stream, device):
        if stream is None:
            try:
                import torch
                return ctypes.c_void_p(torch.cuda.current_stream(device).cuda_stream)
            except Exception:
                return None
        if hasattr(stream, "cuda_stream"):
            return ctypes.c_void_p(stream.cuda_stream)
        return ctypes.c_void_p(int(stream))

    def set_stream(self, stream) -> None:
        check(lib().hq_ctx_set_stream(self.h, self._raw_stream(stream, self.device)))

    def sync(self) -> None:
        check(lib().hq_ctx_sync(self.h))

    def enable_timing(self, on: bool = True) -> None:
        check(lib().hq_ctx_enable_timing(self.h, int(on)))

    def kernel_times(self, max_n: int = 1 << 16) -> List[float]:
        """Durations (ms) of the fused-pipeline launches since the last call."""
        buf = (ctypes.c_float * max_n)()
        n = ctypes.c_int32()
        check(lib().hq_ctx_kernel_times(self.h, buf, max_n, ctypes.byref(n)))
        return list(buf[: min(n.value, max_n)])

    def launches(self) -> int:
        """Cumulative number of kernels launched by this context."""
        n = ctypes.c_int64()
        check(lib().hq_ctx_launches(self.h, ctypes.byref(n)))
        return int(n.value)

    def close(self) -> None:
        if getattr(self, "h", None):
            lib().hq_ctx_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    # -- objects
    def load_columns(self, cols: Dict[str, object], host_copy: Optional[bool] = None,
                     stream: bool = False) -> "Table":
        """stream=True: the host arrays stay where they are (HQ_HOST_STREAM); pipelines over
        the table stream it in blocks (pin them, e.g. torch pinned CPU tensors, to overlap)."""
        return Table.load(self, cols, host_copy, stream)

    @staticmethod
    def _build_desc(d: "BuildDesc", src: "Table", key: int, payload: Sequence[int], preds: Sequence[Pred],
                    expected_rows: int, key2: Optional[int] = None) -> None:
        """key2: second key column of a composite (two-column) join key; it is stored
        as payload word 0, ahead of `payload`."""
        d.src = src.h
        if key2 is not None:
            payload = [key2] + list(payload)
            d.composite = 1
        if len(preds) > MAX_PREDS:
            raise ValueError("too many build predicates")
        d.npreds = len(preds)
        for i, p in enumerate(preds):
            d.preds[i] = p
        d.key_col = key
        d.npayload = len(payload)
        for i, c in enumerate(payload):
            d.payload_cols[i] = c
        d.expected_rows = expected_rows

    def build_hash(self, src: "Table", key: int, payload: Sequence[int] = (), preds: Sequence[Pred] = (),
                   expected_rows: int = 0, key2: Optional[int] = None) -> "Hash":
        d = BuildDesc()
        self._build_desc(d, src, key, payload, preds, expected_rows, key2)
        h = ctypes.c_void_p()
        check(lib().hq_build_hash(self.h, ctypes.byref(d), ctypes.byref(h)))
        return Hash(self, h, keep=[src])

    def build_hashes(self, specs: Sequence[tuple]) -> List["Hash"]:
        """Several builds, one host sync: specs = [(src, key, payload, preds, expected_rows), ...]."""
        n = len(specs)
        ds = (BuildDesc * n)()
        for d, spec in zip(ds, specs):
            self._build_desc(d, *spec)
        hs = (ctypes.c_void_p * n)()
        check(lib().hq_build_hashes(self.h, n, ds, hs))
        return [Hash(self, ctypes.c_void_p(hs[i]), keep=[specs[i][0]]) for i in range(n)]

    def import_hash(self, meta: HashMeta, dev_ptr: int, keep=None) -> "Hash":
        h = ctypes.c_void_p()
        check(lib().hq_hash_import(self.h, ctypes.byref(meta), ctypes.c_void_p(dev_ptr), ctypes.byref(h)))
        return Hash(self, h, keep=[keep])

    # -- prepared queries (CUDA graphs, hq.h "prepared queries")
    def capture_begin(self) -> None:
        check(lib().hq_ctx_capture_begin(self.h))

    def capture_end(self) -> "Graph":
        g = ctypes.c_void_p()
        check(lib().hq_ctx_capture_end(self.h, ctypes.byref(g)))
        return Graph(self, g)

    def capture_abort(self) -> None:
        check(lib().hq_ctx_capture_abort(self.h))

    def gather_faults(self, hashes: Sequence["Hash"], results: Sequence["Result"], dev_out: int) -> None:
        """Enqueue the OR of the hashes' build and the results' pipeline fault words into
        FAULT_WORDS int64 at device address dev_out (no host sync; hq_gather_faults)."""
        hs = (ctypes.c_void_p * max(len(hashes), 1))(*[h.h for h in hashes])
        rs = (ctypes.c_void_p * max(len(results), 1))(*[r.h for r in results])
        check(lib().hq_gather_faults(self.h, hs, len(hashes), rs, len(results), ctypes.c_void_p(dev_out)))

    def pack_hashes(self, hashes: Sequence["Hash"], offs: Sequence[int], dev_dst: int) -> None:
        """Copy the hashes' device views into one device buffer at byte offsets (hq_hash_pack)."""
        hs = (ctypes.c_void_p * max(len(hashes), 1))(*[h.h for h in hashes])
        os_ = (ctypes.c_int64 * max(len(offs), 1))(*[int(o) for o in offs])
        check(lib().hq_hash_pack(self.h, hs, len(hashes), os_, ctypes.c_void_p(dev_dst)))

    def run(self, plan: Plan, keep=(), block_rows: Optional[int] = None) -> "Result":
        """Enqueue a pipeline.  block_rows: batch processing of an HQ_HOST_STREAM fact
        table with this many rows per block (None: the library default)."""
        h = ctypes.c_void_p()
        if block_rows is None:
            check(lib().hq_run_pipeline(self.h, ctypes.byref(plan), ctypes.byref(h)))
        else:
            check(lib().hq_run_pipeline_streamed(self.h, ctypes.byref(plan), int(block_rows), ctypes.byref(h)))
        return Result(self, h, keep=list(keep))


class Graph:
    """A recorded query step (hq_graph): launch() re-executes every recorded kernel and
    leaves the results it finalizes readable until the next launch."""

    def __init__(self, ctx: Context, h):
        self.ctx, self.h = ctx, h

    def launch(self) -> None:
        check(lib().hq_graph_launch(self.ctx.h, self.h))

    def free(self) -> None:
        if self.h:
            lib().hq_graph_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


class Table:
    def __init__(self, ctx: Context, h, nrows: int, names: List[str], keep=None, host_stream: bool = False):
        self.ctx, self.h, self.nrows, self.names, self._keep = ctx, h, nrows, names, keep
        self.host_stream = host_stream

    @classmethod
    def load(cls, ctx: Context, cols: Dict[str, object], host_copy: Optional[bool] = None,
             stream: bool = False) -> "Table":
        """cols: name -> numpy array (host copy) or torch CUDA tensor (borrowed); with
        stream=True, numpy arrays or torch CPU (pinned) tensors that stay on the host."""
        names = list(cols)
        if not names:
            raise ValueError("empty table")
        arrs = list(cols.values())
        is_dev = [hasattr(a, "is_cuda") and a.is_cuda for a in arrs]
        if stream and any(is_dev):
            raise ValueError("stream=True takes host columns")
        arrs = [a.numpy() if stream and hasattr(a, "numpy") else a for a in arrs]  # torch CPU -> zero-copy view
        if any(is_dev) and not all(is_dev):
            raise ValueError("mix of host and device columns")
        dev = all(is_dev)
        if host_copy is None:
            host_copy = not dev
        keep = []
        n = None
        carr = (Column * len(names))()
        for i, (name, a) in enumerate(zip(names, arrs)):
            if dev:
                import torch
                a = a.contiguous()
                dt = {torch.int8: HQ_I8, torch.int32: HQ_I32, torch.int64: HQ_I64}[a.dtype]
                ptr = a.data_ptr()
                ln = a.numel()
            else:
                a = np.ascontiguousarray(a)
                dt = DTYPE_TO_HQ[a.dtype]
                ptr = a.ctypes.data
                ln = a.shape[0]
            keep.append(a)
            n = ln if n is None else n
            if ln != n:
                raise ValueError("columns of different lengths")
            carr[i].name = name.encode()
            carr[i].type = dt
            carr[i].data = ptr
        h = ctypes.c_void_p()
        flags = HQ_HOST_STREAM if stream else (HQ_DEVICE_BORROW if dev else HQ_HOST_COPY)
        check(lib().hq_load_columns(ctx.h, carr, len(names), n, flags, ctypes.byref(h)))
        # host copies are async: keep the host arrays until the next sync (streamed
        # tables: for the table's lifetime)
        return cls(ctx, h, n, names, keep=keep, host_stream=stream)

    def col(self, name: str) -> int:
        return self.names.index(name)

    def column_range(self, name: str):
        """(min, max) of a column (device reduction; syncs).  Empty: min > max."""
        lo, hi = ctypes.c_int64(), ctypes.c_int64()
        check(lib().hq_column_range(self.ctx.h, self.h, self.col(name), ctypes.byref(lo), ctypes.byref(hi)))
        return lo.value, hi.value

    def column_ptr(self, c: int):
        """(device pointer, hq_type) of column c."""
        p = ctypes.c_void_p()
        t = ctypes.c_int32()
        check(lib().hq_table_column(self.h, c, ctypes.byref(p), ctypes.byref(t)))
        return p.value, t.value

    def free(self) -> None:
        if self.h:
            lib().hq_free_table(self.h)
            self.h = None

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


class Hash:
    def __init__(self, ctx: Context, h, keep=None):
        self.ctx, self.h, self._keep = ctx, h, keep

    def info(self) -> HashMeta:
        m = HashMeta()
        check(lib().hq_hash_info(self.ctx.h, self.h, ctypes.byref(m)))
        return m

    def meta(self) -> HashMeta:
        """The table's metadata as the host knows it after the build call (sizes, key and
        payload ranges: exact from the count pass or the cached statistics; nkeys = -1 for
        expected_rows builds), without a sync -- build faults are raised by info() or by
        the finalize of a result that probed the table."""
        return self.device_view()[1]

    def device_view(self):
        p = ctypes.c_void_p()
        m = HashMeta()
        check(lib().hq_hash_device_view(self.h, ctypes.byref(p), ctypes.byref(m)))
        return p.value, m

    def free(self) -> None:
        if self.h:
            lib().hq_free_hash(self.h)
            self.h = None

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


class Result:
    def __init__(self, ctx: Context, h, keep=None):
        self.ctx, self.h, self._keep = ctx, h, keep

    def finalize(self) -> None:
        check(lib().hq_finalize(self.ctx.h, self.h))

    def info(self) -> ResultInfo:
        ri = ResultInfo()
        check(lib().hq_result_info_get(self.ctx.h, self.h, ctypes.byref(ri)))
        return ri

    def fetch(self) -> List[np.ndarray]:
        ri = self.info()
        n = ri.nrows
        outs = [np.empty(max(n, 1), dtype=HQ_TO_DTYPE[ri.types[c]]) for c in range(ri.ncols)]
        ptrs = (ctypes.c_void_p * max(ri.ncols, 1))(*[o.ctypes.data for o in outs])
        got = ctypes.c_int64()
        check(lib().hq_fetch_result(self.ctx.h, self.h, ptrs, n, ctypes.byref(got)))
        return [o[:n] for o in outs]

    def qualifying(self) -> int:
        return int(self.info().qualifying_rows)

    def as_table(self, names: List[str]) -> Table:
        """The result as a table (no host sync when a materialised result of the same
        identity was viewed before: its row count is cached and checked on the device)."""
        h = ctypes.c_void_p()
        check(lib().hq_result_as_table(self.ctx.h, self.h, ctypes.byref(h)))
        n, nc = ctypes.c_int64(), ctypes.c_int32()
        check(lib().hq_table_info(h, ctypes.byref(n), ctypes.byref(nc)))
        return Table(self.ctx, h, int(n.value), names, keep=[self])

    def partials_view(self):
        p = ctypes.c_void_p()
        n = ctypes.c_size_t()
        check(lib().hq_result_partials_view(self.h, ctypes.byref(p), ctypes.byref(n)))
        return p.value, n.value

    def to_partials(self, dev_ptr: int, nbytes: int) -> None:
        """Copy the dense partials into a caller device buffer (hq_result_to_partials)."""
        check(lib().hq_result_to_partials(self.ctx.h, self.h, ctypes.c_void_p(dev_ptr), nbytes))

    def from_partials(self, dev_ptr: int, nbytes: int) -> None:
        """Copy reduced partials back into the result's group table (hq_result_from_partials)."""
        check(lib().hq_result_from_partials(self.ctx.h, self.h, ctypes.c_void_p(dev_ptr), nbytes))

    def free(self) -> None:
        if self.h:
            lib().hq_free_result(self.h)
            self.h = None

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


def raise_faults(words: Sequence[int]) -> None:
    """Raise the HQError a set of gathered (and rank-summed) fault words maps to."""
    arr = (ctypes.c_int64 * FAULT_WORDS)(*[int(w) for w in words])
    check(lib().hq_raise_faults(arr))


# ---- plan construction helpers ----------------------------------------------
_CMP = {"=": EQ, "==": EQ, "!=": NE, "<": LT, "<=": LE, ">": GT, ">=": GE, "between": BETWEEN, "in": IN_BITMAP}


def make_pred(reg: int, cmp, lo=0, hi=0) -> Pred:
    p = Pred()
    p.reg = reg
    p.cmp = _CMP[cmp] if isinstance(cmp, str) else int(cmp)
    if p.cmp == IN_BITMAP:
        bm = [0, 0, 0, 0]
        for v in lo:
            if not 0 <= int(v) < 256:
                raise ValueError("IN-list values must be dictionary codes 0..255")
            bm[int(v) >> 6] |= 1 << (int(v) & 63)
        for i in range(4):
            p.bitmap[i] = bm[i]
    else:
        p.lo = int(lo)
        p.hi = int(hi)
    return p
