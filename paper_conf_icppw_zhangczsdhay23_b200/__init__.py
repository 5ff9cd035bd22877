"""B200-native bucket-aware asynchronous Delta-stepping SSSP (Zhang et al., ICPP-W 2023).

Thin Python binding over the C-ABI library ``libsssp.so`` (``include/sssp.h``):
argument marshalling only -- every step of the SSSP path runs in the sm_100a
kernels behind the ABI. PyTorch is used only for device memory and streams.
The names mirror the C functions (``sssp_graph_create`` ... ``sssp_destroy``);
``Graph`` is a convenience wrapper owning one handle.

There is no CPU fallback: if the shared library is missing this module raises
at import time (build it with ``python -c "import __graft_entry__ as g; g.build()"``).
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("SSSP_LIB") or os.path.join(_HERE, "libsssp.so")  # override: experiments only

if not os.path.exists(LIB_PATH):
    raise ImportError(f"libsssp.so not built at {LIB_PATH}; run __graft_entry__.build() (no CPU fallback exists)")

_lib = ctypes.CDLL(LIB_PATH)

SSSP_OK = 0
SSSP_ERR_INVALID_ARGUMENT = 1
SSSP_ERR_OUT_OF_MEMORY = 2
SSSP_ERR_CUDA = 3
SSSP_ERR_INVALID_STATE = 4
SSSP_ERR_OVERFLOW = 5
SSSP_ERR_INTERNAL = 6
SSSP_WEIGHT_U32 = 0
SSSP_WEIGHT_F32 = 1
SSSP_MEM_HOST = 0
SSSP_MEM_DEVICE = 1
SSSP_PRO_DEGREE = 1
SSSP_PRO_WEIGHT = 2
SSSP_PARAM_RING_SLOTS = 0
SSSP_PARAM_CTAS_PER_SM = 1
SSSP_PARAM_SLOT_CAPACITY = 2
SSSP_PARAM_CLAIM_MAX = 3
SSSP_PARAM_L2_PERSIST = 4
SSSP_PARAM_ADWL = 5
SSSP_PARAM_SYNC = 6
SSSP_PARAM_P2_EDGE_BALANCED = 7
SSSP_PARAM_ADAPTIVE_DELTA = 8
SSSP_PARAM_MULTI_ALIGN = 9
SSSP_PARAM_MULTI_HUB_DELAY = 10
SSSP_PARAM_PULL_SYMMETRIC = 11
SSSP_PARAM_LOCAL_CHASE = 12
SSSP_PARAM_LOCAL_LIMIT = 13
SSSP_PARAM_BF_TAIL = 14
SSSP_BF_TAIL_DEFAULT = 262144

INF_U32 = 0xFFFFFFFF

# Every symbol include/sssp.h declares (checked by tests/test_abi.py).
EXPORTS = (
    "sssp_graph_create", "sssp_reorder", "sssp_reorder_ex", "sssp_run", "sssp_distances",
    "sssp_destroy", "sssp_status_string", "sssp_last_error", "sssp_set_stream", "sssp_run_batch",
    "sssp_get_stats", "sssp_export_csr", "sssp_set_param", "sssp_device_sm_count",
    "sssp_kernel_time", "sssp_get_trace", "sssp_get_profile", "sssp_run_multi", "sssp_multi_stats",
    "sssp_distances_async", "sssp_wait", "sssp_is_symmetric", "sssp_get_samples", "sssp_set_allocator",
)


class sssp_stats(ctypes.Structure):
    _fields_ = [(n, ctypes.c_uint64) for n in (
        "updates", "light_arcs", "heavy_arcs", "vertices_settled", "stale_items", "heavy_vertices",
        "hub_chunks", "bin_thread", "bin_warp", "bin_cta", "buckets", "rescans", "reachable", "levels")] + [
        ("ring_slots", ctypes.c_uint32), ("grid_ctas", ctypes.c_uint32),
        ("run_ms", ctypes.c_float), ("reorder_ms", ctypes.c_float)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


_P, _I64, _I, _D, _U = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int, ctypes.c_double, ctypes.c_uint
_lib.sssp_graph_create.argtypes = [ctypes.POINTER(_P), _I, _I64, _I64, _P, _P, _P, _I, _I, _P]
_lib.sssp_reorder.argtypes = [_P]
_lib.sssp_reorder_ex.argtypes = [_P, _U]
_lib.sssp_run.argtypes = [_P, _I64, _D]
_lib.sssp_distances.argtypes = [_P, _P, _I]
_lib.sssp_destroy.argtypes = [_P]
_lib.sssp_destroy.restype = None
_lib.sssp_status_string.argtypes = [_I]
_lib.sssp_status_string.restype = ctypes.c_char_p
_lib.sssp_last_error.argtypes = []
_lib.sssp_last_error.restype = ctypes.c_char_p
_lib.sssp_set_stream.argtypes = [_P, _P]
_lib.sssp_run_batch.argtypes = [_P, _P, _I64, _D, _P, _I64]
_lib.sssp_run_multi.argtypes = [_P, _P, _I64, _D, _P, _I64]
_lib.sssp_distances_async.argtypes = [_P, _P, _I]
_lib.sssp_wait.argtypes = [_P]
_lib.sssp_is_symmetric.argtypes = [_P, ctypes.POINTER(ctypes.c_int)]
_ALLOC_FN = ctypes.CFUNCTYPE(ctypes.c_void_p, ctypes.c_size_t, ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p)
_FREE_FN = ctypes.CFUNCTYPE(None, ctypes.c_void_p, ctypes.c_size_t, ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p)
_lib.sssp_set_allocator.argtypes = [_ALLOC_FN, _FREE_FN, _P]
_lib.sssp_set_allocator.restype = ctypes.c_int
_lib.sssp_multi_stats.argtypes = [_P, _P, _I64]
_lib.sssp_get_stats.argtypes = [_P, ctypes.POINTER(sssp_stats)]
_lib.sssp_export_csr.argtypes = [_P, _D, _P, _P, _P, _P]
_lib.sssp_set_param.argtypes = [_P, _I, _I64]
_lib.sssp_device_sm_count.argtypes = [_P]
_lib.sssp_kernel_time.argtypes = [_P, ctypes.POINTER(ctypes.c_double), ctypes.POINTER(ctypes.c_int64), _I]
_lib.sssp_kernel_time.restype = _I


class sssp_trace_entry(ctypes.Structure):
    _fields_ = [("t_ns", ctypes.c_uint64), ("which", ctypes.c_uint32), ("cur", ctypes.c_uint32),
                ("tail", ctypes.c_uint32), ("mode", ctypes.c_uint32), ("far_min", ctypes.c_uint32),
                ("pad", ctypes.c_uint32), ("closed_b", ctypes.c_uint32), ("closed_c", ctypes.c_uint32),
                ("t_first", ctypes.c_uint64), ("t_rel", ctypes.c_uint64)]


_lib.sssp_get_trace.argtypes = [_P, _P, _I64, ctypes.POINTER(ctypes.c_int64)]
_lib.sssp_get_trace.restype = _I
_lib.sssp_get_samples.argtypes = [_P, _P, _I64, ctypes.POINTER(ctypes.c_int64)]
_lib.sssp_get_samples.restype = _I
_lib.sssp_get_profile.argtypes = [_P, _P, _I]
_lib.sssp_get_profile.restype = _I
for _n in ("sssp_graph_create", "sssp_reorder", "sssp_reorder_ex", "sssp_run", "sssp_distances",
           "sssp_set_stream", "sssp_run_batch", "sssp_get_stats", "sssp_export_csr", "sssp_set_param",
           "sssp_run_multi", "sssp_multi_stats", "sssp_distances_async", "sssp_wait", "sssp_is_symmetric"):
    getattr(_lib, _n).restype = _I


class SSSPError(RuntimeError):
    def __init__(self, status, where):
        self.status = status
        name = _lib.sssp_status_string(status).decode()
        detail = (_lib.sssp_last_error() or b"").decode()
        super().__init__(f"{where}: {name}: {detail}")


def _check(status, where):
    if status != SSSP_OK:
        raise SSSPError(status, where)


def _ptr(x):
    """Raw pointer + memory kind of a numpy array or torch tensor."""
    if x is None:
        return None, SSSP_MEM_HOST
    if isinstance(x, np.ndarray):
        if not x.flags["C_CONTIGUOUS"]:
            raise ValueError("array must be C-contiguous")
        return x.ctypes.data, SSSP_MEM_HOST
    import torch

    if isinstance(x, torch.Tensor):
        if not x.is_contiguous():
            raise ValueError("tensor must be contiguous")
        return x.data_ptr(), (SSSP_MEM_DEVICE if x.is_cuda else SSSP_MEM_HOST)
    raise TypeError(type(x))


# ---------------------------------------------------------------- C names --
def sssp_graph_create(row, col, w, device=0, stream=None):
    """Create a handle from a CSR given as numpy arrays (host) or CUDA tensors (device)."""
    V = len(row) - 1
    A = int(row[-1]) if isinstance(row, np.ndarray) else int(row[-1].item())
    wdt = w.dtype
    wtype = SSSP_WEIGHT_F32 if str(wdt) in ("float32", "torch.float32") else SSSP_WEIGHT_U32
    if str(wdt) not in ("float32", "torch.float32", "uint32", "torch.uint32", "int32", "torch.int32"):
        raise TypeError(f"weights must be uint32 or float32, got {wdt}")
    rp, k1 = _ptr(row)
    cp, k2 = _ptr(col)
    wp, k3 = _ptr(w)
    if len({k1, k2, k3}) != 1:
        raise ValueError("row/col/w must all be host or all be device")
    h = _P()
    _check(_lib.sssp_graph_create(ctypes.byref(h), int(device), V, A, rp, cp, wp, wtype, k1,
                                  _stream_ptr(stream)), "sssp_graph_create")
    return h


def _stream_ptr(stream):
    if stream is None:
        return None
    return getattr(stream, "cuda_stream", stream)


def sssp_reorder(h):
    _check(_lib.sssp_reorder(h), "sssp_reorder")


def sssp_reorder_ex(h, flags):
    _check(_lib.sssp_reorder_ex(h, int(flags)), "sssp_reorder_ex")


def sssp_run(h, source, delta):
    _check(_lib.sssp_run(h, int(source), float(delta)), "sssp_run")


def sssp_distances(h, out):
    p, kind = _ptr(out)
    _check(_lib.sssp_distances(h, p, kind), "sssp_distances")
    return out


def sssp_distances_async(h, out):
    """Enqueue the output of the last run into ``out`` (pinned host or CUDA
    tensor) on the library's output stream; ``out`` is valid after sssp_wait."""
    p, kind = _ptr(out)
    _check(_lib.sssp_distances_async(h, p, kind), "sssp_distances_async")
    return out


def sssp_wait(h):
    _check(_lib.sssp_wait(h), "sssp_wait")


def sssp_destroy(h):
    _lib.sssp_destroy(h)


def sssp_set_stream(h, stream):
    _check(_lib.sssp_set_stream(h, _stream_ptr(stream)), "sssp_set_stream")


def sssp_run_batch(h, sources, delta, out_dev, ld):
    src = np.ascontiguousarray(sources, dtype=np.int64)
    p, kind = _ptr(out_dev)
    if kind != SSSP_MEM_DEVICE:
        raise ValueError("batch output must be a CUDA tensor")
    _check(_lib.sssp_run_batch(h, src.ctypes.data, len(src), float(delta), p, int(ld)), "sssp_run_batch")


def sssp_run_multi(h, sources, delta, out_dev, ld):
    src = np.ascontiguousarray(sources, dtype=np.int64)
    p, kind = _ptr(out_dev)
    if kind != SSSP_MEM_DEVICE:
        raise ValueError("batch output must be a CUDA tensor")
    _check(_lib.sssp_run_multi(h, src.ctypes.data, len(src), float(delta), p, int(ld)), "sssp_run_multi")


def sssp_multi_stats(h):
    out = np.zeros(7, dtype=np.uint64)
    _check(_lib.sssp_multi_stats(h, out.ctypes.data, 7), "sssp_multi_stats")
    return dict(zip(("updates", "arcs", "expansions", "stale", "split_items", "buckets", "rescans"),
                    (int(x) for x in out)))


def sssp_get_stats(h):
    s = sssp_stats()
    _check(_lib.sssp_get_stats(h, ctypes.byref(s)), "sssp_get_stats")
    return s.as_dict()


def sssp_export_csr(h, V, A, delta, wdtype=np.uint32):
    rowlist = np.empty(2 * V + 1, dtype=np.int64)
    adj = np.empty(max(A, 1), dtype=np.uint32)
    val = np.empty(max(A, 1), dtype=wdtype)
    new2old = np.empty(V, dtype=np.uint32)
    _check(_lib.sssp_export_csr(h, float(delta), rowlist.ctypes.data, adj.ctypes.data, val.ctypes.data,
                                new2old.ctypes.data), "sssp_export_csr")
    return dict(rowlist=rowlist, adj=adj[:A], val=val[:A], new2old=new2old)


def sssp_set_param(h, param, value):
    _check(_lib.sssp_set_param(h, int(param), int(value)), "sssp_set_param")


def sssp_kernel_time(h, reset=False):
    """(total_ms, launches) of the persistent kernel since the last reset."""
    t = ctypes.c_double()
    n = ctypes.c_int64()
    _check(_lib.sssp_kernel_time(h, ctypes.byref(t), ctypes.byref(n), int(reset)), "sssp_kernel_time")
    return t.value, n.value


def sssp_get_trace(h, max_entries=4096):
    """Barrier timeline of the last run: list of dicts (t_us relative to kernel start)."""
    buf = (sssp_trace_entry * max_entries)()
    n = ctypes.c_int64()
    _check(_lib.sssp_get_trace(h, buf, max_entries, ctypes.byref(n)), "sssp_get_trace")
    out = []
    t0 = buf[0].t_ns if n.value else 0
    for i in range(min(n.value, max_entries)):
        e = buf[i]
        out.append(dict(t_us=(e.t_ns - t0) / 1e3, which=e.which, cur=e.cur, tail=e.tail, mode=e.mode,
                        far_min=e.far_min, pad=e.pad, closed_b=e.closed_b, closed_c=e.closed_c,
                        t_first_us=(e.t_first - t0) / 1e3, t_rel_us=(e.t_rel - t0) / 1e3))
    return out


def sssp_get_samples(h, max_entries=16384):
    """Phase-1 claim samples of the last run (diagnostics): list of dicts, t_us relative to
    the first sample."""
    buf = (sssp_trace_entry * max_entries)()
    n = ctypes.c_int64()
    _check(_lib.sssp_get_samples(h, buf, max_entries, ctypes.byref(n)), "sssp_get_samples")
    m = min(n.value, max_entries)
    t0 = min((buf[i].t_ns for i in range(m)), default=0)
    out = []
    for i in range(m):
        b = buf[i]
        if b.which == 101:  # batch record: SM cycles of stage / warp-0 task loop / tail
            out.append(dict(kind="batch", t_us=(b.t_ns - t0) / 1e3, t_ns=b.t_ns, cur=b.cur, tasks=b.tail,
                            tb_tasks=b.mode, ranges=b.far_min, cyc_stage=b.t_first, cyc_task=b.t_rel,
                            cyc_tail=b.pad, cta=b.closed_b, src=b.closed_c))
        else:
            out.append(dict(kind="claim", t_us=(b.t_ns - t0) / 1e3, t_ns=b.t_ns, cur=b.cur, tail=b.tail,
                            claimed=b.mode, pend=b.far_min, pos=b.pad, cta=b.closed_b))
    return out


def sssp_get_profile(h):
    """Cycle accounting of the last run (thread 0 of every persistent CTA)."""
    names = ("claim", "stage", "task", "tail", "barrier", "batches", "tasks",
             "lat_arc", "lat_probe", "lat_atom", "lat_stage", "lat_n", "atoms")
    out = np.zeros(len(names), dtype=np.uint64)
    _check(_lib.sssp_get_profile(h, out.ctypes.data, len(names)), "sssp_get_profile")
    return dict(zip(names, out.tolist()))


_alloc_keep = None  # the ctypes callbacks must outlive every buffer they made


def sssp_set_allocator(alloc=None, free=None):
    """Route the library's device buffers through Python callables:
    alloc(bytes, device, stream) -> int pointer (0 on failure); free(ptr, bytes, device, stream).
    Both None restores cudaMalloc / cudaFree (buffers made by a hook still go back to it)."""
    global _alloc_keep
    if alloc is None and free is None:
        _check(_lib.sssp_set_allocator(_ALLOC_FN(), _FREE_FN(), None), "sssp_set_allocator")
        return
    a = _ALLOC_FN(lambda n, dev, st, ctx: alloc(n, dev, st or 0) or None)
    f = _FREE_FN(lambda ptr, n, dev, st, ctx: free(ptr, n, dev, st or 0))
    _check(_lib.sssp_set_allocator(a, f, None), "sssp_set_allocator")
    _alloc_keep = (_alloc_keep or []) + [(a, f)]


def use_torch_allocator():
    """Back the library's device memory with PyTorch's caching allocator (sssp.h
    sssp_set_allocator): the buffers show up in torch.cuda.memory_allocated()."""
    import torch

    def alloc(n, dev, stream):
        try:
            return torch.cuda.caching_allocator_alloc(n, dev, stream if stream else None)
        except RuntimeError:
            return 0

    def free(ptr, n, dev, stream):
        torch.cuda.caching_allocator_delete(ptr)

    sssp_set_allocator(alloc, free)


def sssp_is_symmetric(h):
    out = ctypes.c_int(0)
    _check(_lib.sssp_is_symmetric(h, ctypes.byref(out)), "sssp_is_symmetric")
    return bool(out.value)


def sssp_device_sm_count(h):
    return int(_lib.sssp_device_sm_count(h))


# ------------------------------------------------------------- wrapper -----
class Graph:
    """Owns one sssp handle. row/col/w: numpy (host) or CUDA tensors."""

    def __init__(self, row, col, w, device=0, stream=None):
        self.V = len(row) - 1
        self.A = int(row[-1]) if isinstance(row, np.ndarray) else int(row[-1].item())
        self.f32 = str(w.dtype) in ("float32", "torch.float32")
        self.device = device
        self.h = sssp_graph_create(row, col, w, device, stream)

    def close(self):
        if self.h:
            sssp_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    def reorder(self, flags=SSSP_PRO_DEGREE | SSSP_PRO_WEIGHT):
        sssp_reorder_ex(self.h, flags)

    def run(self, source, delta):
        sssp_run(self.h, source, delta)

    def distances(self, out=None):
        """Distances in original ids: numpy (host) by default, or into `out`."""
        if out is None:
            out = np.empty(self.V, dtype=np.float32 if self.f32 else np.uint32)
        return sssp_distances(self.h, out)

    def distances_async(self, out):
        """Stream the last run's distances into `out` (pinned host or CUDA tensor)
        while the next run proceeds; read `out` only after wait()."""
        return sssp_distances_async(self.h, out)

    def wait(self):
        sssp_wait(self.h)

    def sssp(self, source, delta, out=None):
        self.run(source, delta)
        return self.distances(out)

    def run_batch(self, sources, delta, out_dev, ld=None):
        sssp_run_batch(self.h, sources, delta, out_dev, ld or self.V)

    def run_multi(self, sources, delta, out_dev, ld=None):
        """NEXT-4: the batch computed 32 sources per persistent launch."""
        sssp_run_multi(self.h, sources, delta, out_dev, ld or self.V)

    def multi_stats(self):
        return sssp_multi_stats(self.h)

    def stats(self):
        return sssp_get_stats(self.h)

    def export_csr(self, delta):
        return sssp_export_csr(self.h, self.V, self.A, delta, np.float32 if self.f32 else np.uint32)

    def set_param(self, param, value):
        sssp_set_param(self.h, param, value)

    def kernel_time(self, reset=False):
        return sssp_kernel_time(self.h, reset)

    def profile(self):
        return sssp_get_profile(self.h)

    def trace(self):
        return sssp_get_trace(self.h)

    def samples(self):
        return sssp_get_samples(self.h)

    def set_stream(self, stream):
        sssp_set_stream(self.h, stream)

    def is_symmetric(self):
        return sssp_is_symmetric(self.h)
