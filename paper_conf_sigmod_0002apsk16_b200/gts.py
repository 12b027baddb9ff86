"""Thin ctypes binding of libgts.so (include/gts.h) -- argument marshalling only.

Every function keeps the C name.  All computation happens in libgts.so's
CUDA kernels; there is no Python or CPU fallback: if the library is missing
this module raises at import, and compute calls without a GPU return
GTS_ECUDA (raised as GtsError).
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "lib", "libgts.so")

if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} is missing: build it with `make` (or __graft_entry__.build()); "
                      "there is no fallback implementation")
_lib = ctypes.CDLL(LIB_PATH)

GTS_OK = 0
GTS_EINVAL, GTS_ENOMEM, GTS_ECUDA, GTS_ENCCL, GTS_EUNSUPPORTED, GTS_EOVERFLOW = -1, -2, -3, -4, -5, -6
GTS_PAGE_SP, GTS_PAGE_LP = 0, 1
GTS_ENTRY_VID32, GTS_ENTRY_PID16_SLOT16 = 0, 1
GTS_STRATEGY_P, GTS_STRATEGY_S, GTS_STRATEGY_S_BCAST = 0, 1, 2
GTS_RESIDENCY_AUTO, GTS_RESIDENT, GTS_STREAMED = 0, 1, 2
GTS_DANGLING_UNIFORM, GTS_DANGLING_DROP = 0, 1
GTS_OUT_HOST, GTS_OUT_DEVICE = 0, 1
GTS_RUN_TIMING = 1
GTS_ROUTE_PEER = 2
# micro-level technique inside each page (gts_run_config.flags bits 8-10; App E, Fig 14)
GTS_MICRO_DEFAULT, GTS_MICRO_EDGE, GTS_MICRO_VERTEX, GTS_MICRO_HYBRID, GTS_MICRO_TILE = 0, 1 << 8, 2 << 8, 3 << 8, 4 << 8
MICRO = {"default": GTS_MICRO_DEFAULT, "edge": GTS_MICRO_EDGE, "vertex": GTS_MICRO_VERTEX,
         "hybrid": GTS_MICRO_HYBRID, "tile": GTS_MICRO_TILE}
GTS_BUILD_DEGREE_ORDER, GTS_BUILD_SYMMETRIC, GTS_BUILD_OWNER_FILTER = 1, 2, 4
GTS_UNREACHED = 0xFFFFFFFF
GTS_OFF = 0xFFFFFFFF

EXPORTED = ["gts_last_error", "gts_version", "gts_build_pages", "gts_plan_pages", "gts_graph_get_stats",
            "gts_graph_pages", "gts_graph_directory", "gts_graph_order", "gts_graph_free", "gts_get_unique_id",
            "gts_context_create", "gts_context_free", "gts_context_evict", "gts_context_set_stream",
            "gts_bfs", "gts_pagerank", "gts_sssp", "gts_wcc", "gts_bc", "gts_partition_pages"]


class GtsError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__(f"gts error {code}: {msg}")
        self.code = code


class PageConfig(ctypes.Structure):
    _fields_ = [(k, ctypes.c_uint32) for k in ("struct_size", "page_bytes", "entry_encoding", "flags", "owner_rank",
                                               "owner_world", "owner_strategy", "reserved")]


class GraphStats(ctypes.Structure):
    _fields_ = [(k, ctypes.c_uint64) for k in ("n", "m", "num_pages", "n_sp", "n_lp", "n_lp_vertices",
                                               "page_bytes", "topo_bytes", "used_bytes", "max_outdeg")] + \
               [(k, ctypes.c_uint32) for k in ("weighted", "entry_encoding", "n_hot", "ordered")] + \
               [("host_page_bytes", ctypes.c_uint64), ("symmetric", ctypes.c_uint32), ("owner_rank", ctypes.c_int32),
                ("owner_world", ctypes.c_uint32), ("owner_strategy", ctypes.c_uint32)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


class RunConfig(ctypes.Structure):
    _fields_ = [(k, ctypes.c_uint32) for k in ("struct_size", "strategy", "residency", "ring_slots",
                                               "batch_pages", "out_location", "flags", "cache_mib",
                                               "virtual_ranks", "sssp_delta", "levels_per_sync", "l2_persist_mib",
                                               "bfs_level_slots", "wcc_sample", "hybrid_deg", "reserved")]

# gts_run_config 1.1 fields settable through the keyword `tune` of the compute calls
TUNABLE = ("sssp_delta", "levels_per_sync", "l2_persist_mib", "bfs_level_slots", "wcc_sample", "hybrid_deg")


class RunStats(ctypes.Structure):
    _fields_ = [(k, ctypes.c_double) for k in ("wall_s", "upload_s", "main_kernel_s", "finish_s", "merge_s",
                                               "h2d_s")] + \
               [(k, ctypes.c_uint64) for k in ("h2d_bytes", "nccl_bytes", "pages_processed", "edges_traversed",
                                               "launches", "main_kernel_launches")] + \
               [(k, ctypes.c_uint32) for k in ("levels_or_iters", "reserved")] + \
               [(k, ctypes.c_uint64) for k in ("cache_hits", "cache_misses", "wa_bytes", "routed_msgs")]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_ if k != "reserved"}


_vp = ctypes.c_void_p
_u64, _u32, _i32 = ctypes.c_uint64, ctypes.c_uint32, ctypes.c_int
_sig = {
    "gts_last_error": (ctypes.c_char_p, []),
    "gts_version": (_i32, []),
    "gts_build_pages": (_i32, [_u64, _u64, _vp, _vp, _vp, ctypes.POINTER(PageConfig), ctypes.POINTER(_vp)]),
    "gts_plan_pages": (_i32, [_u64, _vp, _i32, ctypes.POINTER(PageConfig), ctypes.POINTER(GraphStats)]),
    "gts_graph_get_stats": (_i32, [_vp, ctypes.POINTER(GraphStats)]),
    "gts_graph_pages": (_vp, [_vp]),
    "gts_graph_directory": (_i32, [_vp, _vp, _vp, _vp, _vp, _vp]),
    "gts_graph_order": (_i32, [_vp, _vp]),
    "gts_graph_free": (None, [_vp]),
    "gts_get_unique_id": (_i32, [_vp]),
    "gts_context_create": (_i32, [_i32, _i32, _i32, _vp, ctypes.POINTER(_vp)]),
    "gts_context_free": (None, [_vp]),
    "gts_context_evict": (_i32, [_vp, _vp]),
    "gts_context_set_stream": (_i32, [_vp, _vp]),
    "gts_bfs": (_i32, [_vp, _vp, _u64, ctypes.POINTER(RunConfig), _vp, ctypes.POINTER(RunStats)]),
    "gts_pagerank": (_i32, [_vp, _vp, _u32, ctypes.c_double, _u32, ctypes.POINTER(RunConfig), _vp,
                            ctypes.POINTER(RunStats)]),
    "gts_sssp": (_i32, [_vp, _vp, _u64, ctypes.POINTER(RunConfig), _vp, ctypes.POINTER(RunStats)]),
    "gts_wcc": (_i32, [_vp, _vp, ctypes.POINTER(RunConfig), _vp, ctypes.POINTER(RunStats)]),
    "gts_bc": (_i32, [_vp, _vp, _vp, _u32, ctypes.POINTER(RunConfig), _vp, ctypes.POINTER(RunStats)]),
    "gts_partition_pages": (_i32, [_vp, _u32, _i32, _vp, _vp]),
}
for _name, (_res, _args) in _sig.items():
    _f = getattr(_lib, _name)
    _f.restype = _res
    _f.argtypes = _args


def _check(rc):
    if rc != GTS_OK:
        raise GtsError(rc, _lib.gts_last_error().decode(errors="replace"))


def _np_ptr(a):
    return ctypes.c_void_p(a.ctypes.data) if a is not None else None


def gts_version():
    return _lib.gts_version()


def gts_last_error():
    return _lib.gts_last_error().decode(errors="replace")


def _page_config(page_bytes, entry_encoding, order=False, symmetric=False, owner=None):
    """owner = (rank, world, strategy): build only that rank's pages (GTS_BUILD_OWNER_FILTER)."""
    flags = (GTS_BUILD_DEGREE_ORDER if order else 0) | (GTS_BUILD_SYMMETRIC if symmetric else 0)
    r = w = st = 0
    if owner is not None:
        flags |= GTS_BUILD_OWNER_FILTER
        r, w, st = (int(x) for x in owner)
    return PageConfig(ctypes.sizeof(PageConfig), int(page_bytes), int(entry_encoding), flags, r, w, st, 0)


class Graph:
    """Owner of a gts_graph* (host pages + RVT)."""

    def __init__(self, handle, n, m):
        self._h = handle
        self.n, self.m = n, m

    @property
    def handle(self):
        if self._h is None:
            raise ValueError("graph freed")
        return self._h

    def stats(self):
        st = GraphStats()
        _check(_lib.gts_graph_get_stats(self.handle, ctypes.byref(st)))
        return st.as_dict()

    def pages(self):
        """Copy of the host page bytes this graph holds (uint8; every page in ID order, or with an owner
        filter that rank's pages in ascending ID)."""
        st = self.stats()
        nbytes = st["host_page_bytes"]
        p = _lib.gts_graph_pages(self.handle)
        return np.ctypeslib.as_array((ctypes.c_uint8 * nbytes).from_address(p)).copy() if nbytes else \
            np.zeros(0, np.uint8)

    def directory(self):
        P = self.stats()["num_pages"]
        sv, ns, kd = (np.empty(P, np.uint32) for _ in range(3))
        lf, ll = np.empty(P, np.int64), np.empty(P, np.int64)
        _check(_lib.gts_graph_directory(self.handle, _np_ptr(sv), _np_ptr(ns), _np_ptr(kd), _np_ptr(lf),
                                        _np_ptr(ll)))
        return {"start_vid": sv, "nslots": ns, "kind": kd, "lp_first": lf, "lp_last": ll}

    def order(self):
        """internal_of[v]: internal ID of caller VID v (identity unless built with order=True)."""
        a = np.empty(self.n, np.uint32)
        _check(_lib.gts_graph_order(self.handle, _np_ptr(a)))
        return a

    def free(self):
        if self._h is not None:
            _lib.gts_graph_free(self._h)
            self._h = None

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


def gts_build_pages(row_ptr, col_idx, weights=None, page_bytes=1 << 20, entry_encoding=GTS_ENTRY_VID32, order=False,
                    symmetric=False, owner=None):
    row_ptr = np.ascontiguousarray(row_ptr, dtype=np.uint64)
    col_idx = np.ascontiguousarray(col_idx, dtype=np.uint32)
    if weights is not None:
        weights = np.ascontiguousarray(weights, dtype=np.uint32)
    n = row_ptr.shape[0] - 1
    m = col_idx.shape[0]
    cfg = _page_config(page_bytes, entry_encoding, order, symmetric, owner)
    h = ctypes.c_void_p()
    _check(_lib.gts_build_pages(n, m, _np_ptr(row_ptr), _np_ptr(col_idx), _np_ptr(weights), ctypes.byref(cfg),
                                ctypes.byref(h)))
    return Graph(h, n, 2 * m if symmetric else m)


def gts_plan_pages(row_ptr, weighted=False, page_bytes=1 << 20, entry_encoding=GTS_ENTRY_VID32):
    row_ptr = np.ascontiguousarray(row_ptr, dtype=np.uint64)
    st = GraphStats()
    cfg = _page_config(page_bytes, entry_encoding)
    _check(_lib.gts_plan_pages(row_ptr.shape[0] - 1, _np_ptr(row_ptr), 1 if weighted else 0, ctypes.byref(cfg),
                               ctypes.byref(st)))
    return st.as_dict()


def gts_partition_pages(graph, strategy, world_size):
    P = graph.stats()["num_pages"]
    owner = np.empty(P, np.int32)
    vrange = np.empty(world_size + 1, np.uint64)
    _check(_lib.gts_partition_pages(graph.handle, strategy, world_size, _np_ptr(owner), _np_ptr(vrange)))
    return owner, vrange


def gts_get_unique_id() -> bytes:
    buf = (ctypes.c_uint8 * 128)()
    _check(_lib.gts_get_unique_id(ctypes.cast(buf, ctypes.c_void_p)))
    return bytes(buf)


class Context:
    def __init__(self, handle, device, rank, world_size):
        self._h = handle
        self.device, self.rank, self.world_size = device, rank, world_size

    @property
    def handle(self):
        if self._h is None:
            raise ValueError("context freed")
        return self._h

    def set_stream(self, cuda_stream):
        _check(_lib.gts_context_set_stream(self.handle, ctypes.c_void_p(cuda_stream) if cuda_stream else None))

    def evict(self, graph=None):
        _check(_lib.gts_context_evict(self.handle, graph.handle if graph is not None else None))

    def free(self):
        if self._h is not None:
            _lib.gts_context_free(self._h)
            self._h = None

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


def gts_context_create(device=0, rank=0, world_size=1, unique_id: bytes | None = None):
    h = ctypes.c_void_p()
    uid = None
    if unique_id is not None:
        uid = (ctypes.c_uint8 * 128).from_buffer_copy(unique_id)
    _check(_lib.gts_context_create(device, rank, world_size, ctypes.cast(uid, ctypes.c_void_p) if uid else None,
                                   ctypes.byref(h)))
    return Context(h, device, rank, world_size)


def _run_config(strategy, residency, ring_slots, batch_pages, out_location, timing, cache_mib=0, micro=0,
                virtual_ranks=0, tune=None):
    micro = MICRO[micro] if isinstance(micro, str) else int(micro)
    rc = RunConfig(ctypes.sizeof(RunConfig), strategy, residency, ring_slots, batch_pages, out_location,
                   (GTS_RUN_TIMING if timing else 0) | micro, int(cache_mib), int(virtual_ranks))
    for k, v in (tune or {}).items():
        if k not in TUNABLE:
            raise ValueError(f"unknown tuning field {k}")
        setattr(rc, k, int(v))
    return rc


def _out(out, n, dtype, ctx=None):
    """Host numpy array, or a torch tensor (CUDA on the context's device, or CPU) -> (obj, ptr, location).
    Every buffer must be contiguous, of the result's element size, with >= n elements: libgts writes
    n elements through the pointer."""
    if out is None:
        out = np.empty(n, dtype=dtype)
    isz = np.dtype(dtype).itemsize
    if isinstance(out, np.ndarray):
        if out.dtype != dtype or out.size < n or not out.flags.c_contiguous or not out.flags.writeable:
            raise ValueError(f"output must be a writeable contiguous {dtype} array of >= {n} elements")
        return out, ctypes.c_void_p(out.ctypes.data), GTS_OUT_HOST
    if not (hasattr(out, "data_ptr") and hasattr(out, "numel") and hasattr(out, "element_size")):
        raise TypeError("unsupported output buffer (numpy array or torch tensor)")
    if out.numel() < n or out.element_size() != isz or not out.is_contiguous():
        raise ValueError(f"output tensor must be contiguous, {isz}-byte elements, >= {n} elements")
    if getattr(out, "is_cuda", False):
        if ctx is not None and out.device.index is not None and out.device.index != ctx.device:
            raise ValueError(f"device output is on cuda:{out.device.index}, the context on cuda:{ctx.device}")
        return out, ctypes.c_void_p(out.data_ptr()), GTS_OUT_DEVICE
    return out, ctypes.c_void_p(out.data_ptr()), GTS_OUT_HOST     # pinned/pageable host tensor


def gts_bfs(ctx, graph, src, out=None, strategy=GTS_STRATEGY_P, residency=GTS_RESIDENCY_AUTO, ring_slots=0,
            batch_pages=0, timing=False, cache_mib=0, micro=GTS_MICRO_DEFAULT, virtual_ranks=0, tune=None,
            route_peer=False):
    """Returns (levels, stats dict).  micro: GTS_MICRO_* or "default"/"edge"/"vertex"/"hybrid".
    virtual_ranks=V: run the V-rank job of `strategy` on this GPU.  tune: {gts_run_config 1.1 field: value}."""
    out, ptr, loc = _out(out, graph.n, np.uint32, ctx)
    cfg = _run_config(strategy, residency, ring_slots, batch_pages, loc, timing, cache_mib, micro, virtual_ranks, tune)
    cfg.flags |= GTS_ROUTE_PEER if route_peer else 0
    st = RunStats()
    _check(_lib.gts_bfs(ctx.handle, graph.handle, int(src), ctypes.byref(cfg), ptr, ctypes.byref(st)))
    return out, st.as_dict()


def gts_pagerank(ctx, graph, iters=10, damping=0.85, dangling=GTS_DANGLING_UNIFORM, out=None,
                 strategy=GTS_STRATEGY_P, residency=GTS_RESIDENCY_AUTO, ring_slots=0, batch_pages=0, timing=False,
                 micro=GTS_MICRO_DEFAULT, virtual_ranks=0, tune=None, route_peer=False):
    """route_peer: Strategy-S adds remote updates straight into their owner's WA over peer memory."""
    out, ptr, loc = _out(out, graph.n, np.float32, ctx)
    cfg = _run_config(strategy, residency, ring_slots, batch_pages, loc, timing, 0, micro, virtual_ranks, tune)
    if route_peer:
        cfg.flags |= GTS_ROUTE_PEER
    st = RunStats()
    _check(_lib.gts_pagerank(ctx.handle, graph.handle, int(iters), float(damping), int(dangling),
                             ctypes.byref(cfg), ptr, ctypes.byref(st)))
    return out, st.as_dict()


def gts_sssp(ctx, graph, src, out=None, strategy=GTS_STRATEGY_P, residency=GTS_RESIDENCY_AUTO, ring_slots=0,
             batch_pages=0, timing=False, cache_mib=0, virtual_ranks=0, tune=None, route_peer=False):
    out, ptr, loc = _out(out, graph.n, np.uint32, ctx)
    cfg = _run_config(strategy, residency, ring_slots, batch_pages, loc, timing, cache_mib, 0, virtual_ranks, tune)
    cfg.flags |= GTS_ROUTE_PEER if route_peer else 0
    st = RunStats()
    _check(_lib.gts_sssp(ctx.handle, graph.handle, int(src), ctypes.byref(cfg), ptr, ctypes.byref(st)))
    return out, st.as_dict()


def gts_wcc(ctx, graph, out=None, strategy=GTS_STRATEGY_P, residency=GTS_RESIDENCY_AUTO, ring_slots=0,
            batch_pages=0, timing=False, virtual_ranks=0, tune=None, route_peer=False):
    out, ptr, loc = _out(out, graph.n, np.uint32, ctx)
    cfg = _run_config(strategy, residency, ring_slots, batch_pages, loc, timing, 0, 0, virtual_ranks, tune)
    cfg.flags |= GTS_ROUTE_PEER if route_peer else 0
    st = RunStats()
    _check(_lib.gts_wcc(ctx.handle, graph.handle, ctypes.byref(cfg), ptr, ctypes.byref(st)))
    return out, st.as_dict()


def gts_bc(ctx, graph, sources, out=None, residency=GTS_RESIDENCY_AUTO, ring_slots=0, batch_pages=0, timing=False):
    """Betweenness centrality summed over `sources` (fp64, unnormalised).  Returns (bc, stats)."""
    src = np.ascontiguousarray(sources, dtype=np.uint64)
    out, ptr, loc = _out(out, graph.n, np.float64, ctx)
    cfg = _run_config(GTS_STRATEGY_P, residency, ring_slots, batch_pages, loc, timing)
    st = RunStats()
    _check(_lib.gts_bc(ctx.handle, graph.handle, _np_ptr(src), len(src), ctypes.byref(cfg), ptr, ctypes.byref(st)))
    return out, st.as_dict()
