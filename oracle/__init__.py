"""The GTS oracle -- TEST INFRASTRUCTURE ONLY.

Plain CPU implementations (oracle/oracle.c, fp64 for PageRank and BC;
built single-threaded as liboracle.so and with OpenMP as liboracle_omp.so,
byte-identical outputs) of BFS, PageRank, SSSP, WCC and betweenness centrality over CSR, plus an independent reader
of the slotted-page format.  Only tests/, __graft_entry__.smoke() and
bench.py (cpu_baseline leg and --impl reference) may import this package.
The product path (paper_conf_sigmod_0002apsk16_b200) never imports it and
shares no code with it.

Every function is pinned in tests/test_oracle_*.py; none is "parity
unpinned".
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_OMP_PATH = os.path.join(_HERE, "liboracle_omp.so")
_lib = {}

UNREACHED = 0xFFFFFFFF
DANGLING_UNIFORM = 0
DANGLING_DROP = 1


def build(omp=None):
    """Compile the plain and/or the OpenMP build (omp=None: both)."""
    src = os.path.join(_HERE, "oracle.c")
    if omp in (None, False):
        subprocess.check_call(["gcc", "-O2", "-fPIC", "-shared", "-o", _LIB_PATH, src])
    if omp in (None, True):
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-o", _OMP_PATH, src])


def lib(omp=False):
    """The plain single-threaded build, or (omp=True) the OpenMP build that
    uses OMP_NUM_THREADS (default: all host cores)."""
    if omp not in _lib:
        path = _OMP_PATH if omp else _LIB_PATH
        src = os.path.join(_HERE, "oracle.c")
        if (not os.path.exists(path)) or os.path.getmtime(path) < os.path.getmtime(src):
            build(omp)
        L = ctypes.CDLL(path)
        u64, u32, vp = ctypes.c_uint64, ctypes.c_uint32, ctypes.c_void_p
        L.oracle_bfs.argtypes = [u64, vp, vp, u64, vp]
        L.oracle_bfs.restype = ctypes.c_int
        L.oracle_bfs_levelsync.argtypes = [u64, vp, vp, u64, vp]
        L.oracle_bfs_levelsync.restype = ctypes.c_int
        L.oracle_num_threads.argtypes = []
        L.oracle_num_threads.restype = ctypes.c_int
        L.oracle_pagerank.argtypes = [u64, vp, vp, u32, ctypes.c_double, ctypes.c_int, vp]
        L.oracle_pagerank.restype = ctypes.c_int
        L.oracle_sssp.argtypes = [u64, vp, vp, vp, u64, vp]
        L.oracle_sssp.restype = ctypes.c_int
        L.oracle_wcc.argtypes = [u64, vp, vp, vp]
        L.oracle_wcc.restype = ctypes.c_int
        L.oracle_bc.argtypes = [u64, vp, vp, vp, u64, vp]
        L.oracle_bc.restype = ctypes.c_int
        L.oracle_decode_pages.argtypes = [vp, u64, u64, ctypes.c_int, ctypes.c_int, u64, vp, vp, vp, u64]
        L.oracle_decode_pages.restype = ctypes.c_int64
        _lib[omp] = L
    return _lib[omp]


def num_threads(omp=True):
    """Threads the (OpenMP) build runs with."""
    return int(lib(omp).oracle_num_threads())


def _ptr(a):
    return ctypes.c_void_p(a.ctypes.data) if a is not None else None


def _csr(row_ptr, col):
    row_ptr = np.ascontiguousarray(row_ptr, dtype=np.uint64)
    col = np.ascontiguousarray(col, dtype=np.uint32)
    return row_ptr, col, row_ptr.shape[0] - 1


def bfs(row_ptr, col, src):
    """Hop levels from src over out-edges; UNREACHED = 0xFFFFFFFF."""
    row_ptr, col, n = _csr(row_ptr, col)
    out = np.empty(n, dtype=np.uint32)
    rc = lib().oracle_bfs(n, _ptr(row_ptr), _ptr(col), int(src), _ptr(out))
    if rc:
        raise ValueError(f"oracle_bfs rc={rc}")
    return out


def bfs_levelsync(row_ptr, col, src, omp=True):
    """Same levels as bfs(), level-synchronous; omp=True splits each level over the host cores."""
    row_ptr, col, n = _csr(row_ptr, col)
    out = np.empty(n, dtype=np.uint32)
    rc = lib(omp).oracle_bfs_levelsync(n, _ptr(row_ptr), _ptr(col), int(src), _ptr(out))
    if rc:
        raise ValueError(f"oracle_bfs rc={rc}")
    return out


def pagerank(row_ptr, col, iters=10, damping=0.85, dangling=DANGLING_UNIFORM, omp=False):
    """fp64 pull-order PageRank after `iters` iterations from x0 = 1/n (omp=True: the
    OpenMP build, byte-identical output)."""
    row_ptr, col, n = _csr(row_ptr, col)
    out = np.empty(n, dtype=np.float64)
    rc = lib(omp).oracle_pagerank(n, _ptr(row_ptr), _ptr(col), int(iters), float(damping),
                               1 if dangling == DANGLING_UNIFORM else 0, _ptr(out))
    if rc:
        raise ValueError(f"oracle_pagerank rc={rc}")
    return out


def sssp(row_ptr, col, weights, src):
    """Dijkstra distances (u32; UNREACHED = 0xFFFFFFFF).  Raises OverflowError on >= 2^32-1."""
    row_ptr, col, n = _csr(row_ptr, col)
    w = np.ascontiguousarray(weights, dtype=np.uint32)
    out = np.empty(n, dtype=np.uint32)
    rc = lib().oracle_sssp(n, _ptr(row_ptr), _ptr(col), _ptr(w), int(src), _ptr(out))
    if rc == -6:
        raise OverflowError("distance >= 2^32-1")
    if rc:
        raise ValueError(f"oracle_sssp rc={rc}")
    return out


def wcc(row_ptr, col):
    """Weakly connected components labelled by min VID."""
    row_ptr, col, n = _csr(row_ptr, col)
    out = np.empty(n, dtype=np.uint32)
    rc = lib().oracle_wcc(n, _ptr(row_ptr), _ptr(col), _ptr(out))
    if rc:
        raise ValueError(f"oracle_wcc rc={rc}")
    return out


def bc(row_ptr, col, sources):
    """Brandes betweenness (fp64, unnormalised) accumulated over `sources`."""
    row_ptr, col, n = _csr(row_ptr, col)
    src = np.ascontiguousarray(sources, dtype=np.uint32)
    out = np.empty(n, dtype=np.float64)
    rc = lib().oracle_bc(n, _ptr(row_ptr), _ptr(col), _ptr(src), len(src), _ptr(out))
    if rc:
        raise ValueError(f"oracle_bc rc={rc}")
    return out


def decode_pages(pages, page_bytes, n, m_cap, entry_encoding=0, weighted=False):
    """Rebuild CSR (row_ptr, col, w|None) from slotted-page bytes."""
    pages = np.ascontiguousarray(pages, dtype=np.uint8)
    num_pages = pages.size // page_bytes
    row_ptr = np.empty(n + 1, dtype=np.uint64)
    col = np.empty(max(m_cap, 1), dtype=np.uint32)
    w = np.empty(max(m_cap, 1), dtype=np.uint32) if weighted else None
    m = lib().oracle_decode_pages(_ptr(pages), num_pages, page_bytes, entry_encoding,
                                  1 if weighted else 0, n, _ptr(row_ptr), _ptr(col), _ptr(w), m_cap)
    if m < 0:
        raise ValueError(f"oracle_decode_pages rc={m}")
    return row_ptr, col[:m], (w[:m] if weighted else None)
