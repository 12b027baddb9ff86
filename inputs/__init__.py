"""Seeded synthetic inputs shared by the oracle side and the CUDA side.

Holds none of the GTS method's arithmetic: it only draws graphs (CSR with
sorted rows) and SSSP edge weights.  See inputs/gen.c for the recipes and
DESIGN.md section "Input recipe".
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "libgtsgen.so")
_lib = None

RMAT_ABC = (0.57, 0.19, 0.19)
TWITTER_N = 41_652_230
TWITTER_M = 1_468_365_182
TWITTER_BETA = 1.1
TWITTER_I0 = 271.0
TWITTER_SEED = 2010


def _build():
    src = os.path.join(_HERE, "gen.c")
    subprocess.check_call(["gcc", "-O3", "-march=x86-64-v2", "-fopenmp", "-fPIC", "-shared",
                           "-o", _LIB_PATH, src, "-lm"])


def lib():
    global _lib
    if _lib is None:
        src = os.path.join(_HERE, "gen.c")
        if (not os.path.exists(_LIB_PATH)) or os.path.getmtime(_LIB_PATH) < os.path.getmtime(src):
            _build()
        L = ctypes.CDLL(_LIB_PATH)
        u64p = ctypes.POINTER(ctypes.c_uint64)
        u32p = ctypes.POINTER(ctypes.c_uint32)
        L.gen_rmat.argtypes = [ctypes.c_int, ctypes.c_uint64, ctypes.c_double, ctypes.c_double,
                               ctypes.c_double, ctypes.c_uint64, u64p, u32p]
        L.gen_rmat.restype = ctypes.c_int
        L.gen_rmat_lean.argtypes = L.gen_rmat.argtypes
        L.gen_rmat_lean.restype = ctypes.c_int
        L.gen_twitter_like.argtypes = [ctypes.c_uint64, ctypes.c_uint64, ctypes.c_double,
                                       ctypes.c_double, ctypes.c_uint64, u64p, u32p]
        L.gen_twitter_like.restype = ctypes.c_int
        L.gen_powerlaw_degrees.argtypes = [ctypes.c_uint64, ctypes.c_uint64, ctypes.c_double,
                                           ctypes.c_double, u64p]
        L.gen_powerlaw_degrees.restype = ctypes.c_int
        L.gen_edge_weights.argtypes = [ctypes.c_uint64, u64p, u32p, ctypes.c_uint64, u32p]
        L.gen_edge_weights.restype = None
        L.gen_num_threads.restype = ctypes.c_int
        L.gen_permute_csr.argtypes = [ctypes.c_uint64, u64p, u32p, u32p, u64p, u32p]
        L.gen_permute_csr.restype = ctypes.c_int
        L.gen_indegree_order.argtypes = [ctypes.c_uint64, u64p, u32p, u32p]
        L.gen_indegree_order.restype = ctypes.c_int
        _lib = L
    return _lib


def _p64(a):
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_uint64))


def _p32(a):
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_uint32))


class CSR:
    """A directed multigraph in CSR form (u64 row_ptr[n+1], u32 col[m], optional u32 w[m])."""

    def __init__(self, row_ptr, col, weights=None, name=""):
        self.row_ptr = np.ascontiguousarray(row_ptr, dtype=np.uint64)
        self.col = np.ascontiguousarray(col, dtype=np.uint32)
        self.weights = None if weights is None else np.ascontiguousarray(weights, dtype=np.uint32)
        self.name = name

    @property
    def n(self):
        return int(self.row_ptr.shape[0] - 1)

    @property
    def m(self):
        return int(self.col.shape[0])

    def outdeg(self):
        return np.diff(self.row_ptr).astype(np.uint64)

    def with_weights(self, seed=0x53535350):
        w = edge_weights(self, seed)
        return CSR(self.row_ptr, self.col, w, self.name)

    def __repr__(self):
        return f"CSR({self.name!r}, n={self.n}, m={self.m}, weighted={self.weights is not None})"


def rmat(scale: int, edge_factor: int = 16, abc=RMAT_ABC, seed: int | None = None, lean: bool = False) -> CSR:
    """Unpermuted RMAT (a,b,c) with m = edge_factor * 2^scale; seed defaults to scale.
    lean=True draws the edges twice instead of buffering them (same graph, less memory)."""
    if seed is None:
        seed = scale
    n = 1 << scale
    m = edge_factor * n
    row_ptr = np.empty(n + 1, dtype=np.uint64)
    col = np.empty(m, dtype=np.uint32)
    fn = lib().gen_rmat_lean if lean else lib().gen_rmat
    rc = fn(scale, edge_factor, abc[0], abc[1], abc[2], seed, _p64(row_ptr), _p32(col))
    if rc != 0:
        raise RuntimeError(f"gen_rmat failed rc={rc}")
    return CSR(row_ptr, col, name=f"rmat{scale}")


def twitter_like(n: int = TWITTER_N, m: int = TWITTER_M, beta: float = TWITTER_BETA,
                 i0: float = TWITTER_I0, seed: int = TWITTER_SEED) -> CSR:
    """Twitter-shaped power-law graph."""
    row_ptr = np.empty(n + 1, dtype=np.uint64)
    col = np.empty(m, dtype=np.uint32)
    rc = lib().gen_twitter_like(n, m, beta, i0, seed, _p64(row_ptr), _p32(col))
    if rc != 0:
        raise RuntimeError(f"gen_twitter_like failed rc={rc}")
    return CSR(row_ptr, col, name=f"twitter_like_n{n}")


def indegree_order(g: CSR) -> np.ndarray:
    """new_of_old: rank of each vertex by in-degree (descending, ties by VID)."""
    p = np.empty(g.n, dtype=np.uint32)
    lib().gen_indegree_order(g.n, _p64(g.row_ptr), _p32(g.col), _p32(p))
    return p


def permute(g: CSR, new_of_old: np.ndarray) -> CSR:
    """The same graph with vertex v renamed new_of_old[v] (rows re-sorted)."""
    new_of_old = np.ascontiguousarray(new_of_old, dtype=np.uint32)
    rp = np.empty_like(g.row_ptr)
    col = np.empty_like(g.col)
    rc = lib().gen_permute_csr(g.n, _p64(g.row_ptr), _p32(g.col), _p32(new_of_old), _p64(rp), _p32(col))
    if rc:
        raise RuntimeError(f"gen_permute_csr rc={rc}")
    return CSR(rp, col, None, g.name + "_perm")


def edge_weights(g: CSR, seed: int = 0x53535350) -> np.ndarray:
    w = np.empty(g.m, dtype=np.uint32)
    lib().gen_edge_weights(g.n, _p64(g.row_ptr), _p32(g.col), seed, _p32(w))
    return w


# ------------------------------------------------------------ hand graphs ---

def from_edges(n: int, edges, weights=None, name="") -> CSR:
    """CSR from an explicit edge list; rows sorted by destination (stable for weights)."""
    edges = np.asarray(edges, dtype=np.int64).reshape(-1, 2)
    if weights is not None:
        weights = np.asarray(weights, dtype=np.uint32)
    order = np.lexsort((edges[:, 1], edges[:, 0])) if len(edges) else np.zeros(0, dtype=np.int64)
    e = edges[order]
    counts = np.bincount(e[:, 0], minlength=n) if len(e) else np.zeros(n, dtype=np.int64)
    row_ptr = np.zeros(n + 1, dtype=np.uint64)
    row_ptr[1:] = np.cumsum(counts)
    w = None if weights is None else weights[order]
    return CSR(row_ptr, e[:, 1].astype(np.uint32), w, name)


def path(n):
    return from_edges(n, [(i, i + 1) for i in range(n - 1)], name=f"path{n}")


def cycle(n):
    return from_edges(n, [(i, (i + 1) % n) for i in range(n)], name=f"cycle{n}")


def out_star(k):
    return from_edges(k + 1, [(0, i) for i in range(1, k + 1)], name=f"outstar{k}")


def in_star(k):
    """k leaves, each with one edge to hub 0; the hub has no out-edges."""
    return from_edges(k + 1, [(i, 0) for i in range(1, k + 1)], name=f"instar{k}")


def binary_tree(n):
    return from_edges(n, [((v - 1) // 2, v) for v in range(1, n)], name=f"bintree{n}")


def random_graph(n, m, seed, self_loops=True):
    rng = np.random.default_rng(seed)
    u = rng.integers(0, n, size=m)
    v = rng.integers(0, n, size=m)
    if not self_loops:
        keep = u != v
        u, v = u[keep], v[keep]
    return from_edges(n, np.stack([u, v], axis=1) if len(u) else np.zeros((0, 2)), name=f"rand{n}_{m}_{seed}")
