"""The C-ABI library loads on a CPU-only box and exports every function that
include/gts.h declares; compute calls without a GPU fail loudly (no fallback)."""
import ctypes
import os
import re

import numpy as np
import pytest

import inputs

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    src = open(os.path.join(ROOT, "include", "gts.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(gts_[a-z0-9_]+)\s*\(", src)))


def test_header_symbols_exported():
    import paper_conf_sigmod_0002apsk16_b200 as G
    lib = ctypes.CDLL(G.gts.LIB_PATH)
    names = _declared()
    assert len(names) >= 18
    for name in names:
        assert hasattr(lib, name), name
    assert sorted(G.EXPORTED) == names


def test_version_and_error_string():
    import paper_conf_sigmod_0002apsk16_b200 as G
    assert G.gts_version() == 10000
    with pytest.raises(G.GtsError):
        G.gts_build_pages(np.array([0, 1], np.uint64), np.array([5], np.uint32))
    assert "col_idx" in G.gts_last_error()


def test_no_cpu_fallback():
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    import paper_conf_sigmod_0002apsk16_b200 as G
    with pytest.raises(G.GtsError) as e:
        G.gts_context_create(0)
    assert e.value.code == G.GTS_ECUDA


def test_partition_pages_host_logic():
    import paper_conf_sigmod_0002apsk16_b200 as G
    g = inputs.rmat(14)
    gr = G.gts_build_pages(g.row_ptr, g.col, page_bytes=4096)
    d = gr.directory()
    P = len(d["start_vid"])
    for world in (1, 2, 3, 4, 8):
        owner, _ = G.gts_partition_pages(gr, G.GTS_STRATEGY_P, world)
        assert np.array_equal(owner, np.arange(P) % world)          # h(j) = j mod N
        owner, vr = G.gts_partition_pages(gr, G.GTS_STRATEGY_S, world)
        assert vr[0] == 0 and vr[-1] == g.n and np.all(np.diff(vr.astype(np.int64)) >= 0)
        assert np.all(np.diff(owner) >= 0) and owner.min() >= 0 and owner.max() < world
        # every page's vertex range lies inside its owner's WA range; LP runs never split
        for p in range(P):
            r = owner[p]
            assert vr[r] <= d["start_vid"][p] < vr[r + 1] or (d["nslots"][p] == 0)
            if d["kind"][p] == G.GTS_PAGE_LP:
                assert owner[d["lp_first"][p]] == r == owner[d["lp_last"][p]]
        counts = np.bincount(owner, minlength=world)
        assert counts.max() - counts.min() <= max(3, P // world // 4 + 2)


def test_config_struct_versioning():
    """gts_page_config / gts_run_config carry struct_size so the ABI can grow: a 1.0
    page config (16 bytes, no owner fields) still builds, a struct smaller than the 1.0
    layout is rejected; unknown builder flags are rejected."""
    import paper_conf_sigmod_0002apsk16_b200 as G
    from paper_conf_sigmod_0002apsk16_b200 import gts as B
    g = inputs.rmat(10)
    rp = np.ascontiguousarray(g.row_ptr, np.uint64)
    col = np.ascontiguousarray(g.col, np.uint32)
    h = ctypes.c_void_p()
    cfg = B.PageConfig(16, 4096, 0, 0, 0, 0, 0, 0)
    assert B._lib.gts_build_pages(g.n, g.m, B._np_ptr(rp), B._np_ptr(col), None, ctypes.byref(cfg), ctypes.byref(h)) == 0
    B._lib.gts_graph_free(h)
    cfg = B.PageConfig(8, 4096, 0, 0, 0, 0, 0, 0)
    assert B._lib.gts_build_pages(g.n, g.m, B._np_ptr(rp), B._np_ptr(col), None, ctypes.byref(cfg),
                                  ctypes.byref(h)) == G.GTS_EINVAL
    cfg = B.PageConfig(ctypes.sizeof(B.PageConfig), 4096, 0, 1 << 7, 0, 0, 0, 0)
    assert B._lib.gts_build_pages(g.n, g.m, B._np_ptr(rp), B._np_ptr(col), None, ctypes.byref(cfg),
                                  ctypes.byref(h)) == G.GTS_EINVAL
    assert "flags" in G.gts_last_error()
    assert ctypes.sizeof(B.RunConfig) == 64 and ctypes.sizeof(B.PageConfig) == 32


def test_weighted_record_layout():
    """Weighted records are u32 sz, u32 0, then (adj, w) pairs, 8-byte aligned
    (include/gts.h "Page layout"): checked byte by byte on a hand graph."""
    import paper_conf_sigmod_0002apsk16_b200 as G
    g = inputs.from_edges(3, [(0, 1), (0, 2), (2, 0)], weights=[7, 9, 5])
    gr = G.gts_build_pages(g.row_ptr, g.col, g.weights, page_bytes=256)
    pg = gr.pages()[:256].view(np.uint32)
    # records from offset 0: v0 = [2, 0, (1, 7), (2, 9)], v1 = [0, 0], v2 = [1, 0, (0, 5)]
    assert list(pg[:12]) == [2, 0, 1, 7, 2, 9, 0, 0, 1, 0, 0, 5]
    assert list(pg[-2:]) == [3, 0]                            # footer: nslots, kind = SP
    slots = pg[-8:-2].reshape(3, 2)[::-1]                      # slot_i at end - 8 - 8(i+1): (vid, off)
    assert [tuple(int(v) for v in x) for x in slots] == [(0, 0), (1, 24), (2, 32)]
