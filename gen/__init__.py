"""Seeded synthetic graph workloads (shared input machinery, no SSSP arithmetic).

Thin ctypes wrapper over ``gen/libsssp_gen.so`` (built from ``gen/gen.c``).
Both the oracle side (tests, bench's cpu_baseline) and the CUDA path consume
the CSR produced here; nothing in this module relaxes, buckets or reorders.

Workload recipes (§5.1.2):
  * Kronecker/RMAT: Graph500 A=.57 B=.19 C=.19 D=.05, V=2^scale,
    E=edgefactor*2^scale, Feistel label scramble, self-loops dropped,
    symmetrised.
  * Road-like grid W x H: all horizontal edges, vertical with p=0.2.
  * Weights: u32 U{1..100} or f32 ((x>>8)+1)*2^-24 in (0,1].
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "libsssp_gen.so")
_lib = None


def build(force: bool = False) -> str:
    src = os.path.join(_HERE, "gen.c")
    if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < max(
        os.path.getmtime(src), os.path.getmtime(os.path.join(_HERE, "gen.h"))
    ):
        subprocess.check_call(
            ["gcc", "-O3", "-std=c11", "-fPIC", "-shared", "-pthread", src, "-o", _LIB_PATH]
        )
    return _LIB_PATH


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB_PATH)
        P, I64, U64, I = ctypes.c_void_p, ctypes.c_int64, ctypes.c_uint64, ctypes.c_int
        lib.gen_rand64.restype = U64
        lib.gen_rand64.argtypes = [U64, U64, U64]
        lib.gen_scramble.restype = ctypes.c_uint32
        lib.gen_scramble.argtypes = [ctypes.c_uint32, I, U64]
        lib.gen_kronecker_edges.argtypes = [I, I64, U64, I, P, P, I]
        lib.gen_grid_edges.restype = I64
        lib.gen_grid_edges.argtypes = [I64, I64, ctypes.c_double, U64, P, P, P]
        lib.gen_weights_u32.argtypes = [I64, P, U64, ctypes.c_uint32, ctypes.c_uint32, P, I]
        lib.gen_weights_f32.argtypes = [I64, P, U64, P, I]
        lib.gen_csr_rows.restype = I64
        lib.gen_csr_rows.argtypes = [I64, I64, P, P, I, P, I]
        lib.gen_csr_fill.argtypes = [I64, I64, P, P, P, I, P, P, P, I]
        lib.gen_sample_sources.restype = I64
        lib.gen_sample_sources.argtypes = [I64, P, I64, U64, P]
        _lib = lib
    return _lib


def _ptr(a):
    return None if a is None else a.ctypes.data


def _nthreads(n):
    return int(n) if n else (os.cpu_count() or 1)


@dataclass
class Graph:
    """CSR graph: row int64[V+1], col uint32[A], w uint32|float32[A]."""

    V: int
    row: np.ndarray
    col: np.ndarray
    w: np.ndarray
    m: int  # undirected input edges (GTEPS numerator)
    name: str = ""

    @property
    def A(self) -> int:
        return int(self.row[-1])

    @property
    def wtype(self) -> str:
        return "f32" if self.w.dtype == np.float32 else "u32"


def csr_from_edges(V, src, dst, w, symmetrize=True, nthreads=None, m=None, name=""):
    """Build a deterministic CSR from an edge list (self-loops dropped).

    Each adjacency is ordered by (dst, weight bits) ascending."""
    lib = _load()
    src = np.ascontiguousarray(src, dtype=np.uint32)
    dst = np.ascontiguousarray(dst, dtype=np.uint32)
    w = np.ascontiguousarray(w)
    if w.dtype not in (np.uint32, np.float32):
        raise TypeError("weights must be uint32 or float32")
    E = len(src)
    row = np.zeros(V + 1, dtype=np.int64)
    nt = _nthreads(nthreads)
    A = lib.gen_csr_rows(V, E, _ptr(src), _ptr(dst), int(symmetrize), _ptr(row), nt)
    col = np.empty(A, dtype=np.uint32)
    wout = np.empty(A, dtype=w.dtype)
    lib.gen_csr_fill(V, E, _ptr(src), _ptr(dst), _ptr(w.view(np.uint32)), int(symmetrize),
                     _ptr(row), _ptr(col), _ptr(wout.view(np.uint32)), nt)
    return Graph(V, row, col, wout, int(E if m is None else m), name)


def _weights(n, eid, seed, weights, lo, hi, nt):
    lib = _load()
    if weights == "u32":
        w = np.empty(n, dtype=np.uint32)
        lib.gen_weights_u32(n, _ptr(eid), seed, lo, hi, _ptr(w), nt)
    elif weights == "f32":
        w = np.empty(n, dtype=np.float32)
        lib.gen_weights_f32(n, _ptr(eid), seed, _ptr(w), nt)
    else:
        raise ValueError(weights)
    return w


def kronecker_edges(scale, edgefactor=16, seed=1, scramble=True, nthreads=None):
    lib = _load()
    E = edgefactor << scale
    src = np.empty(E, dtype=np.uint32)
    dst = np.empty(E, dtype=np.uint32)
    lib.gen_kronecker_edges(scale, E, seed, int(scramble), _ptr(src), _ptr(dst), _nthreads(nthreads))
    return src, dst


def kronecker(scale, edgefactor=16, seed=1, weights="u32", lo=1, hi=100, symmetrize=True,
              scramble=True, nthreads=None):
    """Graph500 Kronecker graph, seeded, symmetrised."""
    nt = _nthreads(nthreads)
    src, dst = kronecker_edges(scale, edgefactor, seed, scramble, nt)
    w = _weights(len(src), None, seed, weights, lo, hi, nt)
    g = csr_from_edges(1 << scale, src, dst, w, symmetrize, nt, m=len(src),
                       name=f"kron-s{scale}-ef{edgefactor}-{weights}-seed{seed}")
    return g


def grid(W, H, p=0.2, seed=2, weights="u32", lo=1, hi=100, nthreads=None):
    """Road-like W x H grid (row-major ids), symmetrised."""
    lib = _load()
    cap = H * (W - 1) + (H - 1) * W
    src = np.empty(max(cap, 1), dtype=np.uint32)
    dst = np.empty(max(cap, 1), dtype=np.uint32)
    eid = np.empty(max(cap, 1), dtype=np.uint64)
    n = lib.gen_grid_edges(W, H, p, seed, _ptr(src), _ptr(dst), _ptr(eid))
    src, dst, eid = src[:n], dst[:n], eid[:n]
    nt = _nthreads(nthreads)
    w = _weights(n, eid, seed, weights, lo, hi, nt)
    return csr_from_edges(W * H, src, dst, w, True, nt, m=n, name=f"grid-{W}x{H}-p{p}-{weights}-seed{seed}")


def sample_sources(g: Graph, n: int, seed: int = 7) -> np.ndarray:
    """n distinct seeded sources with degree >= 1."""
    lib = _load()
    out = np.empty(n, dtype=np.int64)
    k = lib.gen_sample_sources(g.V, _ptr(g.row), n, seed, _ptr(out))
    return out[:k]


def rand64(seed, stream, counter):
    return int(_load().gen_rand64(seed, stream, counter))


def scramble(x, scale, seed):
    return int(_load().gen_scramble(x, scale, seed))


# Named workloads of BASELINE.json "configs". Delta per config is the
# best of a B200 sweep (tools/ab.py --deltas, profiles/r01_summary.md); C3 keeps
# the paper's 0.1, flat within 0.1-0.15.
CONFIGS = {
    "C1": dict(kind="kron", scale=16, edgefactor=16, seed=1, weights="u32", delta=64),
    "C2": dict(kind="grid", W=4894, H=4894, p=0.2, seed=2, weights="u32", delta=6400),
    "C3": dict(kind="kron", scale=22, edgefactor=16, seed=3, weights="f32", delta=0.1),
    "C4": dict(kind="kron", scale=24, edgefactor=16, seed=4, weights="u32", delta=16),
    "C5": dict(kind="kron", scale=26, edgefactor=16, seed=5, weights="u32", delta=16),
}


def make_config(name, nthreads=None, **override):
    c = dict(CONFIGS[name])
    c.update(override)
    if c["kind"] == "kron":
        return kronecker(c["scale"], c["edgefactor"], c["seed"], c["weights"], nthreads=nthreads)
    return grid(c["W"], c["H"], c["p"], c["seed"], c["weights"], nthreads=nthreads)
