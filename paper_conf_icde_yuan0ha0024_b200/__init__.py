"""Python binding of libtdfs.so -- the B200 hot path of T-DFS (Yuan et al., ICDE 2024).

Argument marshalling only: every step of the matching path (edge tasks, queue,
timeout split, paged stacks, Eq. (1) intersection) runs in the CUDA kernels behind
the C-ABI declared in ``include/tdfs.h``.  PyTorch is used for device memory
(workspace, output buffers) and streams.  There is no CPU fallback: if the
compiled library is missing, importing this package raises.

The functions keep the C names (``tdfs_load_graph``, ``tdfs_plan_query``,
``tdfs_count``, ``tdfs_enumerate`` ...).
"""
from __future__ import annotations

import ctypes
import os
from typing import Optional, Sequence, Tuple, Union

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_PKG, "libtdfs.so")

if not os.path.exists(LIB_PATH):
    raise ImportError(f"libtdfs.so not found at {LIB_PATH}: build it first "
                      "(python -m paper_conf_icde_yuan0ha0024_b200.build or __graft_entry__.build()); "
                      "there is no CPU fallback")

_lib = ctypes.CDLL(LIB_PATH)

# ----------------------------------------------------------------- constants
TDFS_OK = 0
STATUS = {0: "TDFS_OK", 1: "TDFS_E_INVALID_ARG", 2: "TDFS_E_GRAPH_FORMAT", 3: "TDFS_E_ID_RANGE",
          4: "TDFS_E_QUERY_DISCONNECTED", 5: "TDFS_E_QUERY_TOO_LARGE", 6: "TDFS_E_LABEL_RANGE", 7: "TDFS_E_OOM",
          8: "TDFS_E_STACK_EXHAUSTED", 9: "TDFS_E_OUTPUT_OVERFLOW", 10: "TDFS_E_CUDA", 11: "TDFS_E_WORKSPACE"}
for _code, _name in STATUS.items():
    globals()[_name] = _code
TDFS_MAX_K = 8
TDFS_MEM_HOST_COPY = 0
TDFS_MEM_DEVICE_BORROW = 1
TDFS_GRAPH_VALIDATE = 1
TDFS_GRAPH_NORMALIZE = 2
TDFS_GRAPH_DEGREE_ORDER = 4
TDFS_RUN_STATS = 1
TDFS_RUN_TRACE = 2
TDFS_RUN_NO_REUSE = 4
TDFS_RUN_NO_SHORTCUT = 8
TDFS_RUN_NO_HUB_BITMAP = 16
TDFS_RUN_NO_LEAF_STAGE = 32
TDFS_RUN_ARRAY_STACKS = 128
TDFS_RUN_NO_RANGE_TASKS = 256
TDFS_SHARD_ROUND_ROBIN = 0
TDFS_SHARD_DEGREE_BALANCED = 1
TDFS_SHARD_BLOCKED = 2
TDFS_SHARD_BLOCK_EDGES = 1024
TDFS_COUNT_INVALID = (1 << 64) - 1


class TdfsError(RuntimeError):
    def __init__(self, status: int, detail: str):
        super().__init__(f"{STATUS.get(status, status)}: {detail}")
        self.status = status
        self.detail = detail


# ----------------------------------------------------------------- structs
class tdfs_csr(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int64), ("nnz", ctypes.c_int64), ("offs", ctypes.c_void_p), ("adj", ctypes.c_void_p),
                ("label", ctypes.c_void_p), ("mem", ctypes.c_int32), ("flags", ctypes.c_uint32),
                ("hub_bitmap_bytes", ctypes.c_int64)]


class tdfs_plan_opts(ctypes.Structure):
    _fields_ = [("order", ctypes.POINTER(ctypes.c_int32)), ("constraints", ctypes.POINTER(ctypes.c_int32)),
                ("n_constraints", ctypes.c_int32)]


class tdfs_run_opts(ctypes.Structure):
    _fields_ = [("tau_ns", ctypes.c_int64), ("chunk", ctypes.c_int32), ("queue_ints", ctypes.c_int64),
                ("page_bytes", ctypes.c_int32), ("page_table_entries", ctypes.c_int32),
                ("pool_bytes", ctypes.c_int64), ("blocks", ctypes.c_int32), ("warps_per_block", ctypes.c_int32),
                ("shard_rank", ctypes.c_int32), ("shard_world", ctypes.c_int32), ("flags", ctypes.c_uint32),
                ("shard_policy", ctypes.c_int32), ("reserved_", ctypes.c_int32), ("shared_cursor", ctypes.c_void_p)]


class tdfs_stats(ctypes.Structure):
    _fields_ = [("nodes_per_level", ctypes.c_uint64 * (TDFS_MAX_K + 1)), ("adj_bytes", ctypes.c_uint64),
                ("tasks_enqueued", ctypes.c_uint64), ("tasks_dequeued", ctypes.c_uint64),
                ("timeouts", ctypes.c_uint64), ("queue_full", ctypes.c_uint64), ("pages_used", ctypes.c_uint64),
                ("edges_scanned", ctypes.c_uint64), ("edges_filtered_in", ctypes.c_uint64),
                ("chunks_fetched", ctypes.c_uint64), ("kernel_ms", ctypes.c_float), ("grid_blocks", ctypes.c_int32),
                ("warps_per_block", ctypes.c_int32), ("page_table_entries", ctypes.c_int32), ("pad_", ctypes.c_int32),
                ("pool_pages", ctypes.c_uint64), ("stream_bytes", ctypes.c_uint64),
                ("warp_exit_first_ns", ctypes.c_uint64), ("warp_exit_mean_ns", ctypes.c_uint64),
                ("warp_exit_last_ns", ctypes.c_uint64)]

    def as_dict(self) -> dict:
        d = {f: getattr(self, f) for f, _ in self._fields_ if f not in ("nodes_per_level", "pad_")}
        d["nodes_per_level"] = [int(x) for x in self.nodes_per_level]
        return d


_vp = ctypes.c_void_p
_i32p = ctypes.POINTER(ctypes.c_int32)
_i64p = ctypes.POINTER(ctypes.c_int64)
_u64p = ctypes.POINTER(ctypes.c_uint64)

# Exported symbols of include/tdfs.h and include/tdfs_test.h with their ctypes signatures.
SIGNATURES = {
    "tdfs_status_string": (ctypes.c_char_p, [ctypes.c_int]),
    "tdfs_last_error": (ctypes.c_char_p, []),
    "tdfs_abi_version": (ctypes.c_int, []),
    "tdfs_load_graph": (ctypes.c_int, [ctypes.POINTER(tdfs_csr), ctypes.c_int, _vp, ctypes.POINTER(_vp)]),
    "tdfs_load_edges": (ctypes.c_int, [ctypes.c_int64, ctypes.c_int64, _vp, _vp, _vp, ctypes.c_uint32, ctypes.c_int64,
                                       ctypes.c_int, _vp, ctypes.POINTER(_vp)]),
    "tdfs_graph_info": (ctypes.c_int, [_vp, _i64p, _i64p, _i64p, _i32p]),
    "tdfs_graph_device_arrays": (ctypes.c_int, [_vp, ctypes.POINTER(_vp), ctypes.POINTER(_vp), ctypes.POINTER(_vp)]),
    "tdfs_free_graph": (None, [_vp]),
    "tdfs_plan_query": (ctypes.c_int, [ctypes.c_int32, ctypes.c_int32, _i32p, _i32p, ctypes.POINTER(tdfs_plan_opts),
                                       ctypes.POINTER(_vp)]),
    "tdfs_plan_order": (ctypes.c_int, [_vp, _i32p]),
    "tdfs_plan_constraints": (ctypes.c_int, [_vp, _i32p, ctypes.c_int32, _i32p]),
    "tdfs_plan_aut_size": (ctypes.c_int, [_vp, _i64p]),
    "tdfs_plan_k": (ctypes.c_int, [_vp, _i32p]),
    "tdfs_free_plan": (None, [_vp]),
    "tdfs_run_opts_default": (None, [ctypes.POINTER(tdfs_run_opts)]),
    "tdfs_workspace_bytes": (ctypes.c_size_t, [_vp, _vp, ctypes.POINTER(tdfs_run_opts)]),
    "tdfs_count": (ctypes.c_int, [_vp, _vp, ctypes.POINTER(tdfs_run_opts), _vp, ctypes.c_size_t, _vp, _vp, _u64p,
                                  ctypes.POINTER(tdfs_stats)]),
    "tdfs_enumerate": (ctypes.c_int, [_vp, _vp, ctypes.POINTER(tdfs_run_opts), _vp, ctypes.c_size_t, _vp, _vp,
                                      ctypes.c_uint64, _u64p, ctypes.POINTER(tdfs_stats)]),
    "tdfs_workspace_status": (ctypes.c_int, [_vp, _vp]),
    "tdfs_enumerate_stream": (ctypes.c_int, [_vp, _vp, ctypes.POINTER(tdfs_run_opts), _vp, ctypes.c_size_t, _vp, _vp,
                                             ctypes.c_uint64, _vp, _vp, _u64p]),
    "tdfs_enumerate_to_file": (ctypes.c_int, [_vp, _vp, ctypes.POINTER(tdfs_run_opts), _vp, ctypes.c_size_t, _vp,
                                              _vp, ctypes.c_uint64, ctypes.c_char_p, _u64p]),
    "tdfs_partition_edges": (ctypes.c_int, [ctypes.c_int64, ctypes.c_int64, _vp, _vp, ctypes.c_int32, ctypes.c_int32,
                                            _vp]),
    "tdfs_shared_cursor_create": (ctypes.c_int, [ctypes.c_int, ctypes.POINTER(_vp), _vp]),
    "tdfs_shared_cursor_open": (ctypes.c_int, [ctypes.c_int, _vp, ctypes.POINTER(_vp)]),
    "tdfs_shared_cursor_reset": (ctypes.c_int, [_vp, _vp]),
    "tdfs_shared_cursor_close": (ctypes.c_int, [_vp, ctypes.c_int]),
    "tdfs_test_queue": (ctypes.c_int, [ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_int64, ctypes.c_uint64,
                                       ctypes.c_int64, _i32p, _i32p, _i64p, _i64p]),
    "tdfs_test_paged_write": (ctypes.c_int, [ctypes.c_int, ctypes.c_int, ctypes.c_int64, ctypes.c_uint32, _i32p,
                                             _i32p, _i32p, _i32p, _i32p]),
    "tdfs_test_count_trace": (ctypes.c_int, [_vp, _vp, ctypes.POINTER(tdfs_run_opts), _vp, ctypes.c_size_t, _vp,
                                             _i32p, ctypes.c_int64, _i64p, _u64p]),
}
for _name, (_res, _args) in SIGNATURES.items():
    _f = getattr(_lib, _name)
    _f.restype = _res
    _f.argtypes = _args


def last_error() -> str:
    s = _lib.tdfs_last_error()
    return s.decode() if s else ""


def _check(rc: int, allow=()) -> int:
    if rc != TDFS_OK and rc not in allow:
        raise TdfsError(rc, last_error())
    return rc


def tdfs_abi_version() -> int:
    return _lib.tdfs_abi_version()


def tdfs_status_string(s: int) -> str:
    return _lib.tdfs_status_string(s).decode()


# ----------------------------------------------------------------- handles
def _torch():
    import torch
    return torch


def _stream_ptr(stream, device: int) -> Optional[int]:
    if stream is None:
        torch = _torch()
        return torch.cuda.current_stream(device).cuda_stream
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


class GraphHandle:
    """Owns a tdfs_graph* (freed on garbage collection)."""

    def __init__(self, ptr: int, device: int, keepalive=None):
        self.ptr = ptr
        self.device = device
        self._keep = keepalive

    def info(self) -> dict:
        n, m, dmax, nl = ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int32()
        _check(_lib.tdfs_graph_info(self.ptr, ctypes.byref(n), ctypes.byref(m), ctypes.byref(dmax), ctypes.byref(nl)))
        return {"n": n.value, "m": m.value, "dmax": dmax.value, "nlabels": nl.value}

    def free(self):
        if self.ptr:
            _lib.tdfs_free_graph(self.ptr)
            self.ptr = None

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


class PlanHandle:
    def __init__(self, ptr: int):
        self.ptr = ptr

    @property
    def k(self) -> int:
        k = ctypes.c_int32()
        _check(_lib.tdfs_plan_k(self.ptr, ctypes.byref(k)))
        return k.value

    def order(self):
        out = (ctypes.c_int32 * self.k)()
        _check(_lib.tdfs_plan_order(self.ptr, out))
        return list(out)

    def constraints(self):
        n = ctypes.c_int32()
        buf = (ctypes.c_int32 * 128)()
        _check(_lib.tdfs_plan_constraints(self.ptr, buf, 64, ctypes.byref(n)))
        return [(buf[2 * i], buf[2 * i + 1]) for i in range(n.value)]

    def aut_size(self) -> int:
        a = ctypes.c_int64()
        _check(_lib.tdfs_plan_aut_size(self.ptr, ctypes.byref(a)))
        return a.value

    def __del__(self):
        try:
            if self.ptr:
                _lib.tdfs_free_plan(self.ptr)
                self.ptr = None
        except Exception:
            pass


# ----------------------------------------------------------------- graph loading
def tdfs_load_graph(offs, adj, label=None, device: int = 0, stream=None, validate: bool = False,
                    normalize: bool = False, hub_bitmap_bytes: int = 0, degree_order: bool = False) -> GraphHandle:
    """Load a CSR.  numpy arrays -> HOST_COPY; torch CUDA tensors -> DEVICE_BORROW (kept alive by the handle)."""
    flags = (TDFS_GRAPH_VALIDATE if validate else 0) | (TDFS_GRAPH_NORMALIZE if normalize else 0) | \
        (TDFS_GRAPH_DEGREE_ORDER if degree_order else 0)
    keep = None
    if hasattr(offs, "is_cuda") and offs.is_cuda:
        torch = _torch()
        assert offs.dtype == torch.int64 and adj.dtype == torch.int32
        assert label is None or label.dtype == torch.uint8
        offs, adj = offs.contiguous(), adj.contiguous()
        label = None if label is None else label.contiguous()
        c = tdfs_csr(offs.numel() - 1, adj.numel(), offs.data_ptr(), adj.data_ptr(),
                     None if label is None else label.data_ptr(), TDFS_MEM_DEVICE_BORROW, flags, hub_bitmap_bytes)
        keep = (offs, adj, label)
        device = offs.device.index or 0
    else:
        offs = np.ascontiguousarray(offs, dtype=np.int64)
        adj = np.ascontiguousarray(adj, dtype=np.int32)
        label = None if label is None else np.ascontiguousarray(label, dtype=np.uint8)
        c = tdfs_csr(offs.shape[0] - 1, adj.shape[0], offs.ctypes.data, adj.ctypes.data,
                     None if label is None else label.ctypes.data, TDFS_MEM_HOST_COPY, flags, hub_bitmap_bytes)
    out = _vp()
    _check(_lib.tdfs_load_graph(ctypes.byref(c), device, _stream_ptr(stream, device), ctypes.byref(out)))
    return GraphHandle(out.value, device, keep)


def tdfs_load_edges(n: int, edges, label=None, device: int = 0, stream=None, hub_bitmap_bytes: int = 0,
                    degree_order: bool = False) -> GraphHandle:
    """Load an undirected edge list ((m, 2) int array, host) -- normalised by the library."""
    e = np.ascontiguousarray(np.asarray(edges, dtype=np.int32).reshape(-1, 2))
    src = np.ascontiguousarray(e[:, 0])
    dst = np.ascontiguousarray(e[:, 1])
    lab = None if label is None else np.ascontiguousarray(label, dtype=np.uint8)
    out = _vp()
    _check(_lib.tdfs_load_edges(int(n), e.shape[0], src.ctypes.data, dst.ctypes.data,
                                None if lab is None else lab.ctypes.data,
                                TDFS_GRAPH_DEGREE_ORDER if degree_order else 0, int(hub_bitmap_bytes), device,
                                _stream_ptr(stream, device), ctypes.byref(out)))
    return GraphHandle(out.value, device)


# ----------------------------------------------------------------- planning
def tdfs_plan_query(k: int, qedges: Sequence[Tuple[int, int]], qlabel: Optional[Sequence[int]] = None,
                    order: Optional[Sequence[int]] = None,
                    constraints: Union[str, Sequence[Tuple[int, int]]] = "auto") -> PlanHandle:
    qe = (ctypes.c_int32 * max(1, 2 * len(qedges)))(*[int(x) for e in qedges for x in e])
    ql = None if qlabel is None else (ctypes.c_int32 * k)(*[int(x) for x in qlabel])
    po = tdfs_plan_opts()
    keep = []
    if order is not None:
        oa = (ctypes.c_int32 * k)(*[int(x) for x in order])
        keep.append(oa)
        po.order = oa
    if constraints == "auto":
        po.n_constraints = -1
    elif constraints in ("none", None) or len(constraints) == 0:
        po.n_constraints = 0
    else:
        ca = (ctypes.c_int32 * (2 * len(constraints)))(*[int(x) for c in constraints for x in c])
        keep.append(ca)
        po.constraints = ca
        po.n_constraints = len(constraints)
    out = _vp()
    _check(_lib.tdfs_plan_query(int(k), len(qedges), qe, ql, ctypes.byref(po), ctypes.byref(out)))
    return PlanHandle(out.value)


def plan_from_query(q, order=None, constraints="auto") -> PlanHandle:
    """Plan a tdfs_inputs.Query-like object (k, edges, labels)."""
    return tdfs_plan_query(q.k, q.edges, q.labels, order=order, constraints=constraints)


# ----------------------------------------------------------------- running
def default_opts(**kw) -> tdfs_run_opts:
    o = tdfs_run_opts()
    _lib.tdfs_run_opts_default(ctypes.byref(o))
    for key, val in kw.items():
        if key == "tau_ms":
            o.tau_ns = -1 if val is None or val == float("inf") else int(val * 1e6)
            continue
        if not hasattr(o, key):
            raise KeyError(key)
        setattr(o, key, val)
    return o


def tdfs_workspace_bytes(g: GraphHandle, p: PlanHandle, opts: Optional[tdfs_run_opts] = None) -> int:
    opts = opts or default_opts()
    n = _lib.tdfs_workspace_bytes(g.ptr, p.ptr, ctypes.byref(opts))
    if n == 0:
        raise TdfsError(TDFS_E_INVALID_ARG, last_error())
    return n


class Workspace:
    """Caller-owned device workspace (a torch uint8 tensor), grown on demand."""

    def __init__(self, device: int = 0):
        self.device = device
        self.t = None

    def get(self, nbytes: int):
        torch = _torch()
        if self.t is None or self.t.numel() < nbytes:
            self.t = None
            self.t = torch.empty(int(nbytes), dtype=torch.uint8, device=f"cuda:{self.device}")
        return self.t


_default_ws = {}


def _ws_for(g: GraphHandle, nbytes: int, workspace):
    if workspace is None:
        workspace = _default_ws.setdefault(g.device, Workspace(g.device))
    if isinstance(workspace, Workspace):
        return workspace.get(nbytes)
    return workspace


def tdfs_count(g: GraphHandle, p: PlanHandle, opts: Optional[tdfs_run_opts] = None, workspace=None, stream=None,
               d_count=None, sync: bool = True, stats: bool = False):
    """Count matches.  sync=True returns the int count (and a stats dict if stats=True).
    sync=False enqueues the job on `stream` and writes the count to `d_count`
    (a 1-element uint64/int64 CUDA tensor), returning None."""
    opts = opts or default_opts()
    nbytes = tdfs_workspace_bytes(g, p, opts)
    ws = _ws_for(g, nbytes, workspace)
    st = _stream_ptr(stream, g.device)
    h = ctypes.c_uint64(0)
    s = tdfs_stats() if stats else None
    dptr = None if d_count is None else d_count.data_ptr()
    rc = _lib.tdfs_count(g.ptr, p.ptr, ctypes.byref(opts), ws.data_ptr(), ws.numel(), st, dptr,
                         ctypes.byref(h) if (sync or stats) else None, ctypes.byref(s) if stats else None)
    _check(rc)
    if not (sync or stats):
        return None
    if stats:
        return int(h.value), s.as_dict()
    return int(h.value)


def tdfs_enumerate(g: GraphHandle, p: PlanHandle, cap: int, opts: Optional[tdfs_run_opts] = None, workspace=None,
                   stream=None, out=None, stats: bool = False):
    """Enumerate matches: returns (tuples as an (min(total,cap), k) int32 numpy array, total, overflow[, stats])."""
    torch = _torch()
    opts = opts or default_opts()
    k = p.k
    nbytes = tdfs_workspace_bytes(g, p, opts)
    ws = _ws_for(g, nbytes, workspace)
    if out is None:
        out = torch.empty(max(1, cap) * k, dtype=torch.int32, device=f"cuda:{g.device}")
    st = _stream_ptr(stream, g.device)
    tot = ctypes.c_uint64(0)
    s = tdfs_stats() if stats else None
    rc = _lib.tdfs_enumerate(g.ptr, p.ptr, ctypes.byref(opts), ws.data_ptr(), ws.numel(), st, out.data_ptr(),
                             int(cap), ctypes.byref(tot), ctypes.byref(s) if stats else None)
    _check(rc, allow=(TDFS_E_OUTPUT_OVERFLOW,))
    n = min(int(tot.value), int(cap))
    arr = out[: n * k].view(n, k).cpu().numpy()
    res = (arr, int(tot.value), rc == TDFS_E_OUTPUT_OVERFLOW)
    return res + (s.as_dict(),) if stats else res


def tdfs_enumerate_chunks(g: GraphHandle, p: PlanHandle, chunk_cap: int, opts: Optional[tdfs_run_opts] = None,
                          workspace=None, stream=None):
    """Enumerate every match of this caller's shard as a generator of (tuples, total_so_far), tuples
    an (n <= chunk_cap, k) int32 numpy array indexed by query vertex id.

    Marshalling only: one tdfs_enumerate_stream job (the kernel writes into a device ring of
    8 * ceil(chunk_cap / 8) tuples drained by the library) runs on a helper thread; its sink hands
    each drained chunk to this generator through a bounded queue, so a slow consumer back-pressures
    the kernel (its warps wait for ring space) instead of buffering without bound."""
    import queue
    import threading

    if chunk_cap < 1:
        raise TdfsError(TDFS_E_INVALID_ARG, "chunk_cap must be >= 1")
    ring_cap = 8 * max(1, -(-chunk_cap // 8))
    q: "queue.Queue" = queue.Queue(maxsize=2)
    stop = threading.Event()
    res = {}

    def sink(arr):
        for i in range(0, arr.shape[0], chunk_cap):
            while True:
                if stop.is_set():
                    return True
                try:
                    q.put(arr[i:i + chunk_cap], timeout=0.1)
                    break
                except queue.Full:
                    continue
        return False

    def run():
        try:
            res["total"] = tdfs_enumerate_stream(g, p, sink, ring_cap, opts, workspace, stream)
        except BaseException as e:  # noqa: BLE001 -- re-raised in the generator
            res["error"] = e
        finally:
            q.put(None)

    th = threading.Thread(target=run, daemon=True)
    th.start()
    done = 0
    try:
        while True:
            item = q.get()
            if item is None:
                break
            done += item.shape[0]
            yield item, done
    finally:
        stop.set()
        while th.is_alive():
            try:
                q.get(timeout=0.1)
            except queue.Empty:
                pass
        th.join()
    if "error" in res:
        raise res["error"]
    if res.get("total") != done:
        raise TdfsError(TDFS_E_CUDA, f"streamed {done} tuples, job total {res.get('total')}")


TUPLE_SINK = ctypes.CFUNCTYPE(ctypes.c_int, ctypes.POINTER(ctypes.c_int32), ctypes.c_uint64, ctypes.c_int32,
                              ctypes.c_void_p)


def _ring(g: GraphHandle, k: int, ring_cap: int):
    torch = _torch()
    if ring_cap < 8 or ring_cap % 8:
        raise TdfsError(TDFS_E_INVALID_ARG, "ring_cap must be a positive multiple of 8")
    return torch.empty(ring_cap * k, dtype=torch.int32, device=f"cuda:{g.device}")


def tdfs_enumerate_stream(g: GraphHandle, p: PlanHandle, sink, ring_cap: int = 1 << 20,
                          opts: Optional[tdfs_run_opts] = None, workspace=None, stream=None) -> int:
    """Stream every match (NEXT-2): sink(tuples) receives (n, k) int32 numpy arrays (a copy), indexed
    by query vertex id; returning True stops delivery.  Returns the exact total."""
    opts = opts or default_opts()
    k = p.k
    ring = _ring(g, k, ring_cap)
    ws = _ws_for(g, tdfs_workspace_bytes(g, p, opts), workspace)
    err = []

    def _cb(ptr, n, kk, user):
        try:
            arr = np.ctypeslib.as_array(ptr, shape=(int(n) * int(kk),)).reshape(int(n), int(kk)).copy()
            return 1 if sink(arr) else 0
        except Exception as e:  # noqa: BLE001 -- re-raised after the call
            err.append(e)
            return 1

    cb = TUPLE_SINK(_cb)
    tot = ctypes.c_uint64(0)
    rc = _lib.tdfs_enumerate_stream(g.ptr, p.ptr, ctypes.byref(opts), ws.data_ptr(), ws.numel(),
                                    _stream_ptr(stream, g.device), ring.data_ptr(), int(ring_cap),
                                    ctypes.cast(cb, ctypes.c_void_p), None, ctypes.byref(tot))
    if err:
        raise err[0]
    _check(rc)
    return int(tot.value)


def tdfs_enumerate_to_file(g: GraphHandle, p: PlanHandle, path: str, ring_cap: int = 1 << 20,
                           opts: Optional[tdfs_run_opts] = None, workspace=None, stream=None) -> int:
    """Every match of this shard (opts.shard_rank / shard_world: a rank-local file) into `path`:
    raw int32 rows of k ids (query-vertex order).  Returns the exact total."""
    opts = opts or default_opts()
    ring = _ring(g, p.k, ring_cap)
    ws = _ws_for(g, tdfs_workspace_bytes(g, p, opts), workspace)
    tot = ctypes.c_uint64(0)
    _check(_lib.tdfs_enumerate_to_file(g.ptr, p.ptr, ctypes.byref(opts), ws.data_ptr(), ws.numel(),
                                       _stream_ptr(stream, g.device), ring.data_ptr(), int(ring_cap),
                                       os.fsencode(path), ctypes.byref(tot)))
    return int(tot.value)


def tdfs_workspace_status(workspace, stream=None, device: int = 0) -> int:
    return _check(_lib.tdfs_workspace_status(workspace.data_ptr(), _stream_ptr(stream, device)))


# ----------------------------------------------------------------- multi-GPU helpers
def tdfs_partition_edges(offs, adj, world: int, policy: int = TDFS_SHARD_ROUND_ROBIN) -> np.ndarray:
    """Owner rank of every directed edge (host CSR numpy arrays) under a shard policy (tdfs.h)."""
    offs = np.ascontiguousarray(offs, dtype=np.int64)
    adj = np.ascontiguousarray(adj, dtype=np.int32)
    owner = np.empty(max(1, adj.shape[0]), dtype=np.int32)
    _check(_lib.tdfs_partition_edges(offs.shape[0] - 1, adj.shape[0], offs.ctypes.data, adj.ctypes.data,
                                     int(world), int(policy), owner.ctypes.data))
    return owner[: adj.shape[0]]


class SharedCursor:
    """A uint64 chunk cursor in one rank's device memory, mapped by the others through CUDA IPC
    (tdfs_shared_cursor_*; cross-GPU dynamic balancing)."""

    def __init__(self, device: int, handle: Optional[bytes] = None):
        self.device = device
        p = _vp()
        if handle is None:
            buf = ctypes.create_string_buffer(64)
            _check(_lib.tdfs_shared_cursor_create(device, ctypes.byref(p), buf))
            self.handle = buf.raw
            self.opened = 0
        else:
            self.handle = bytes(handle)
            _check(_lib.tdfs_shared_cursor_open(device, ctypes.create_string_buffer(self.handle, 64),
                                                ctypes.byref(p)))
            self.opened = 1
        self.ptr = p.value

    def reset(self, stream=None):
        _check(_lib.tdfs_shared_cursor_reset(self.ptr, _stream_ptr(stream, self.device)))

    def close(self):
        if self.ptr:
            _check(_lib.tdfs_shared_cursor_close(self.ptr, self.opened))
            self.ptr = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


# ----------------------------------------------------------------- test hooks
def tdfs_test_queue(mode: int, tasks: np.ndarray, cap_tasks: int, n_warps: int = 1, ticket_base: int = 0,
                    device: int = 0):
    t = np.ascontiguousarray(np.asarray(tasks, dtype=np.int32).reshape(-1, 3))
    out = np.zeros_like(t) if t.shape[0] else np.zeros((1, 3), np.int32)
    n_out, n_enq = ctypes.c_int64(), ctypes.c_int64()
    _check(_lib.tdfs_test_queue(device, mode, n_warps, cap_tasks, ticket_base, t.shape[0],
                                t.ctypes.data_as(_i32p), out.ctypes.data_as(_i32p), ctypes.byref(n_out),
                                ctypes.byref(n_enq)))
    return out[: n_out.value], n_enq.value


def tdfs_test_paged_write(page_bytes: int, start_pos: int, valid_mask: int = 0xFFFFFFFF, device: int = 0):
    page = (ctypes.c_int32 * 32)()
    off = (ctypes.c_int32 * 32)()
    nnew, first, rb = ctypes.c_int32(), ctypes.c_int32(), ctypes.c_int32()
    _check(_lib.tdfs_test_paged_write(device, page_bytes, start_pos, valid_mask, page, off, ctypes.byref(nnew),
                                      ctypes.byref(first), ctypes.byref(rb)))
    return {"page": list(page), "offset": list(off), "new_pages": nnew.value, "first_lane_on_new_page": first.value,
            "readback_ok": rb.value}


def tdfs_test_count_trace(g: GraphHandle, p: PlanHandle, opts: tdfs_run_opts, cap: int = 1 << 20, workspace=None,
                          stream=None):
    nbytes = tdfs_workspace_bytes(g, p, opts)
    ws = _ws_for(g, nbytes, workspace)
    tr = np.zeros((cap, 3), dtype=np.int32)
    nt = ctypes.c_int64()
    cnt = ctypes.c_uint64()
    _check(_lib.tdfs_test_count_trace(g.ptr, p.ptr, ctypes.byref(opts), ws.data_ptr(), ws.numel(),
                                      _stream_ptr(stream, g.device), tr.ctypes.data_as(_i32p), cap,
                                      ctypes.byref(nt), ctypes.byref(cnt)))
    return int(cnt.value), tr[: min(nt.value, cap)], int(nt.value)
