"""CPU oracle for the SSSP hot path -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s cpu_baseline /
``--impl reference`` leg may import this package. The product path never does.
It wraps ``oracle/liboracle.so`` (plain C, ``oracle/oracle.c``), which shares no
code with the CUDA path. See ``oracle/oracle.h`` for the definitions followed
and the PAPER.md passages they cite.

Every function here is pinned by ``tests/test_oracle_pins.py`` against values
the paper prints (Fig. 1, Fig. 4), closed forms and brute force.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lib = None

INF_U32 = 0xFFFFFFFF


def build(force: bool = False) -> str:
    src = os.path.join(_HERE, "oracle.c")
    hdr = os.path.join(_HERE, "oracle.h")
    if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < max(
        os.path.getmtime(src), os.path.getmtime(hdr)
    ):
        # -ffp-contract=off: no FMA contraction; binary32 adds stay single RN ops.
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-ffp-contract=off", "-fno-fast-math",
                               "-fPIC", "-shared", src, "-o", _LIB_PATH, "-lm"])
    return _LIB_PATH


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB_PATH)
        P, I64, I, D = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int, ctypes.c_double
        for name in ("oracle_dijkstra_u32", "oracle_dijkstra_f32"):
            getattr(lib, name).restype = I
            getattr(lib, name).argtypes = [I64, P, P, P, I64, P]
        for name in ("oracle_bellman_ford_u32", "oracle_bellman_ford_f32"):
            getattr(lib, name).restype = I64
            getattr(lib, name).argtypes = [I64, P, P, P, I64, P]
        lib.oracle_floyd_warshall_u32.restype = I
        lib.oracle_floyd_warshall_u32.argtypes = [I64, P, P, P, P]
        lib.oracle_certificate_u32.restype = I64
        lib.oracle_certificate_u32.argtypes = [I64, P, P, P, I64, P]
        lib.oracle_pro_reorder.restype = I
        lib.oracle_pro_reorder.argtypes = [I64, P, P, P, P, P, P, P, P]
        lib.oracle_pro_rowlist.restype = None
        lib.oracle_pro_rowlist.argtypes = [I64, P, P, I, D, P]
        lib.oracle_bucket_histogram.restype = I64
        lib.oracle_bucket_histogram.argtypes = [I64, P, I, D, P, I64]
        _lib = lib
    return _lib


def _c(a, dtype):
    return np.ascontiguousarray(a, dtype=dtype)


def _csr(row, col, w):
    row = _c(row, np.int64)
    col = _c(col, np.uint32)
    w = np.ascontiguousarray(w)
    if w.dtype not in (np.uint32, np.float32):
        raise TypeError("weights must be uint32 or float32")
    return row, col, w


def dijkstra(row, col, w, src):
    """Exact SSSP distances (u32 -> uint32 with INF=0xFFFFFFFF; f32 -> float32, inf)."""
    row, col, w = _csr(row, col, w)
    V = len(row) - 1
    lib = _load()
    if w.dtype == np.uint32:
        out = np.empty(V, dtype=np.uint32)
        rc = lib.oracle_dijkstra_u32(V, row.ctypes.data, col.ctypes.data, w.ctypes.data, int(src), out.ctypes.data)
    else:
        out = np.empty(V, dtype=np.float32)
        rc = lib.oracle_dijkstra_f32(V, row.ctypes.data, col.ctypes.data, w.ctypes.data, int(src), out.ctypes.data)
    if rc == 5:
        raise OverflowError("u32 distance overflow")
    if rc != 0:
        raise ValueError(f"oracle_dijkstra rc={rc}")
    return out


def bellman_ford(row, col, w, src):
    row, col, w = _csr(row, col, w)
    V = len(row) - 1
    lib = _load()
    if w.dtype == np.uint32:
        out = np.empty(V, dtype=np.uint32)
        r = lib.oracle_bellman_ford_u32(V, row.ctypes.data, col.ctypes.data, w.ctypes.data, int(src), out.ctypes.data)
        if r < 0:
            raise OverflowError("u32 distance overflow")
    else:
        out = np.empty(V, dtype=np.float32)
        lib.oracle_bellman_ford_f32(V, row.ctypes.data, col.ctypes.data, w.ctypes.data, int(src), out.ctypes.data)
    return out


def floyd_warshall(row, col, w):
    """All-pairs distances (u32 weights only), uint64 matrix, UINT64_MAX = unreachable."""
    row, col, w = _csr(row, col, w)
    if w.dtype != np.uint32:
        raise TypeError("Floyd-Warshall oracle is integer-only")
    V = len(row) - 1
    D = np.empty((V, V), dtype=np.uint64)
    rc = _load().oracle_floyd_warshall_u32(V, row.ctypes.data, col.ctypes.data, w.ctypes.data, D.ctypes.data)
    if rc != 0:
        raise ValueError("floyd_warshall rc=%d" % rc)
    return D


def certificate(row, col, w, src, dist):
    """-1 if dist is a valid shortest-path certificate (u32, weights >= 1), else offending vertex."""
    row, col, w = _csr(row, col, w)
    dist = _c(dist, np.uint32)
    V = len(row) - 1
    return int(_load().oracle_certificate_u32(V, row.ctypes.data, col.ctypes.data, w.ctypes.data,
                                              int(src), dist.ctypes.data))


def pro_reorder(row, col, w):
    """Property-driven reordering (PAPER §4.1, Fig. 4).

    Returns dict(new2old, old2new, row, adj, val) with val in the weight dtype."""
    row, col, w = _csr(row, col, w)
    V = len(row) - 1
    A = int(row[-1])
    wb = w.view(np.uint32)
    new2old = np.empty(V, dtype=np.uint32)
    old2new = np.empty(V, dtype=np.uint32)
    new_row = np.empty(V + 1, dtype=np.int64)
    adj = np.empty(max(A, 1), dtype=np.uint32)
    val = np.empty(max(A, 1), dtype=np.uint32)
    _load().oracle_pro_reorder(V, row.ctypes.data, col.ctypes.data, wb.ctypes.data, new2old.ctypes.data,
                               old2new.ctypes.data, new_row.ctypes.data, adj.ctypes.data, val.ctypes.data)
    return dict(new2old=new2old, old2new=old2new, row=new_row, adj=adj[:A], val=val[:A].view(w.dtype))


def pro_rowlist(new_row, val, delta):
    """Interleaved (start, heavy) row list + end, 2V+1 entries (Fig. 4c)."""
    new_row = _c(new_row, np.int64)
    val = np.ascontiguousarray(val)
    V = len(new_row) - 1
    out = np.empty(2 * V + 1, dtype=np.int64)
    wtype = 0 if val.dtype == np.uint32 else 1
    vb = val.view(np.uint32) if len(val) else np.zeros(1, np.uint32)
    _load().oracle_pro_rowlist(V, new_row.ctypes.data, vb.ctypes.data, wtype, float(delta), out.ctypes.data)
    return out


def bucket_histogram(dist, delta, nb=4096):
    dist = np.ascontiguousarray(dist)
    wtype = 0 if dist.dtype == np.uint32 else 1
    db = dist.view(np.uint32)
    counts = np.zeros(nb, dtype=np.int64)
    n = _load().oracle_bucket_histogram(len(db), db.ctypes.data, wtype, float(delta), counts.ctypes.data, nb)
    return counts[: min(n, nb)]


def adaptive_delta(C, T, delta0, reading="A", lo=0.25, hi=4.0):
    """Bucket widths of the adaptive Delta variant (NEXT-1), PAPER Eq. (1)-(2)
     step by step, reading R7 for the garbled bars:

        eps_i = 0                                                   i = 0, 1
        eps_i = |C_{i-2} - C_{i-1}| / (C_{i-2} + C_{i-1})
                * (T_{i-2} - T_{i-1}) / (T_{i-2} + T_{i-1}) * Delta_0   i >= 2   (1)
        Delta_i = Delta_{i-1} + eps_i                                        (2)

    C_i / T_i: converged vertices / threads of bucket i. Reading
    "B" takes the Fig. 6 text instead (bucket k ends at 25(k+1) + sum eps,
    P:1033-1037, i.e. Delta_i = Delta_0 + eps_i). Delta_i is clamped to
    [lo, hi] * Delta_0 (our reading; the paper states no bound). A zero
    denominator gives eps_i = 0. Returns [Delta_0, ..., Delta_n] for the
    n = len(C) closed buckets (Delta_i is known once bucket i-1 closes)."""
    assert len(C) == len(T)
    deltas = [float(delta0)]
    for i in range(1, len(C) + 1):
        eps = 0.0
        if i >= 2:
            c2, c1, t2, t1 = float(C[i - 2]), float(C[i - 1]), float(T[i - 2]), float(T[i - 1])
            if c2 + c1 > 0 and t2 + t1 > 0:
                eps = abs(c2 - c1) / (c2 + c1) * ((t2 - t1) / (t2 + t1)) * delta0
        prev = deltas[-1] if reading == "A" else float(delta0)
        deltas.append(min(max(prev + eps, lo * delta0), hi * delta0))
    return deltas
