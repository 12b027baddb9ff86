"""Page builder (gts_build_pages) -- CPU tests, no GPU needed.

Pins: Fig 1 example (T-A, tests/golden/fig1_example.json), App A record-ID
arithmetic (T-B), RVT START_VIDs of Fig 12 (T-C), Table 3 page counts (T-E,
tests/golden/table3_pages.json) and the exact round trip decode(build(CSR)) ==
CSR through the oracle's independent page reader.
"""
import json
import os

import numpy as np
import pytest

import inputs
import oracle
import paper_conf_sigmod_0002apsk16_b200 as G

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _fig1_graph():
    spec = json.load(open(os.path.join(GOLD, "fig1_example.json")))
    n = spec["n"]
    edges = [(0, 1), (0, 2), (1, 0), (1, 2), (2, 0), (2, 1), (2, 3), (3, 2)] + [(3, v) for v in range(4, 100)]
    return spec, inputs.from_edges(n, edges)


def _u32(b, off):
    return int(np.frombuffer(b[off:off + 4].tobytes(), dtype=np.uint32)[0])


def test_fig1_example_structure():
    spec, g = _fig1_graph()
    pb = spec["page_bytes"]
    ex = spec["expect"]
    gr = G.gts_build_pages(g.row_ptr, g.col, page_bytes=pb)
    st = gr.stats()
    d = gr.directory()
    pages = gr.pages().reshape(-1, pb)
    assert list(d["start_vid"][:4]) == ex["rvt_start_vid_prefix"]
    assert d["kind"][0] == G.GTS_PAGE_SP and d["nslots"][0] == 3
    assert list(d["kind"][1:3]) == [G.GTS_PAGE_LP] * ex["v3_lp_pages"]
    assert st["n_lp"] == ex["v3_lp_pages"] and st["n_lp_vertices"] == 1
    assert list(d["lp_first"][1:3]) == [1, 1] and list(d["lp_last"][1:3]) == [2, 2]
    assert d["lp_first"][0] == -1
    # SP0: records packed from offset 0 (40 B), slots from the end (24 B)
    sp0 = pages[0]
    assert _u32(sp0, pb - 8) == 3 and _u32(sp0, pb - 4) == G.GTS_PAGE_SP
    offs = [_u32(sp0, pb - 8 - 8 * (i + 1) + 4) for i in range(3)]
    vids = [_u32(sp0, pb - 8 - 8 * (i + 1)) for i in range(3)]
    assert vids == ex["sp0_vertices"] and offs == [0, 12, 24]
    assert offs[-1] + 4 + 4 * 3 == ex["sp0_record_bytes"]
    assert [_u32(sp0, o) for o in offs] == [2, 2, 3]
    # LP1/LP2: v3's 97 neighbours split 57 + 40; footer total_deg 97, chunk_idx 0/1
    for c, lp in enumerate(pages[1:3]):
        assert _u32(lp, 0) == ex["v3_lp_chunk_lengths"][c]
        assert _u32(lp, pb - 16) == 97 and _u32(lp, pb - 12) == c
        assert _u32(lp, pb - 8) == 1 and _u32(lp, pb - 4) == G.GTS_PAGE_LP
        assert _u32(lp, pb - 24) == 3 and _u32(lp, pb - 20) == 0
    lp1 = pages[1]
    assert _u32(lp1, 4) == 2          # first ADJLIST entry of v3 is r2 -> v2


def test_appendix_a_physical_ids():
    """App A: r2 = (ADJ_PID 0, ADJ_OFF 2) -> VID = RVT[0].START_VID + 2 = 2."""
    spec, g = _fig1_graph()
    pb = spec["page_bytes"]
    gr = G.gts_build_pages(g.row_ptr, g.col, page_bytes=pb, entry_encoding=G.GTS_ENTRY_PID16_SLOT16)
    lp1 = gr.pages().reshape(-1, pb)[1]
    e = _u32(lp1, 4)
    a = spec["expect"]["appendix_a_rid"]
    assert (e >> 16, e & 0xFFFF) == (a["adj_pid"], a["adj_off"])
    sv = gr.directory()["start_vid"]
    assert sv[e >> 16] + (e & 0xFFFF) == a["vid"]
    # the whole graph decodes back through RVT arithmetic
    rp, col, _ = oracle.decode_pages(gr.pages(), pb, g.n, g.m, entry_encoding=1)
    assert np.array_equal(rp, g.row_ptr) and np.array_equal(col, g.col)


@pytest.mark.parametrize("pb", [256, 4096, 65536, 1 << 20])
@pytest.mark.parametrize("maker", ["rmat12", "rmat16", "twitter", "rand", "weighted"])
def test_round_trip(maker, pb):
    if maker == "rmat12":
        g = inputs.rmat(12)
    elif maker == "rmat16":
        g = inputs.rmat(16)
    elif maker == "twitter":
        g = inputs.twitter_like(n=50000, m=400000)
    elif maker == "rand":
        g = inputs.random_graph(3000, 20000, 4)
    else:
        g = inputs.rmat(12).with_weights()
    if pb == 256 and g.m > 100000:
        pytest.skip("256 B pages only for the small graphs")
    gr = G.gts_build_pages(g.row_ptr, g.col, g.weights, page_bytes=pb)
    rp, col, w = oracle.decode_pages(gr.pages(), pb, g.n, g.m, weighted=g.weights is not None)
    assert np.array_equal(rp, g.row_ptr)
    assert np.array_equal(col, g.col)
    if g.weights is not None:
        assert np.array_equal(w, g.weights)
    st = gr.stats()
    d = gr.directory()
    # invariants: START_VID monotone, VID ranges tile [0, n), LP runs are single vertices
    sv, ns = d["start_vid"].astype(np.int64), d["nslots"].astype(np.int64)
    assert np.all(np.diff(sv) >= 0)
    sp = d["kind"] == G.GTS_PAGE_SP
    covered = np.zeros(g.n, dtype=np.int64)
    for s, k in zip(sv[sp], ns[sp]):
        covered[s:s + k] += 1
    lp_v = np.unique(sv[~sp])
    covered[lp_v] += 1
    assert np.all(covered == 1)
    assert st["num_pages"] == st["n_sp"] + st["n_lp"]
    assert st["used_bytes"] <= st["topo_bytes"]
    plan = G.gts_plan_pages(g.row_ptr, weighted=g.weights is not None, page_bytes=pb)
    assert plan["num_pages"] == st["num_pages"] and plan["n_lp"] == st["n_lp"]


def test_multi_edges_self_loops_zero_degree():
    g = inputs.from_edges(6, [(0, 0), (0, 0), (0, 3), (2, 2), (5, 1), (5, 1), (5, 1)])
    gr = G.gts_build_pages(g.row_ptr, g.col, page_bytes=256)
    rp, col, _ = oracle.decode_pages(gr.pages(), 256, g.n, g.m)
    assert np.array_equal(rp, g.row_ptr) and np.array_equal(col, g.col)


def test_vertex_spanning_many_lps():
    k = 5000   # reversed out-star: one vertex of out-degree k -> ceil(k / 57) LPs at 256 B
    g = inputs.out_star(k)
    gr = G.gts_build_pages(g.row_ptr, g.col, page_bytes=256)
    st = gr.stats()
    assert st["n_lp"] == -(-k // 57) and st["n_lp_vertices"] == 1
    rp, col, _ = oracle.decode_pages(gr.pages(), 256, g.n, g.m)
    assert np.array_equal(col, g.col)


def test_table3_rmat27_page_counts():
    spec = json.load(open(os.path.join(GOLD, "table3_pages.json")))["rmat27"]
    s = spec["scale"]
    n = 1 << s
    m = spec["edge_factor"] * n
    k = np.bitwise_count(np.arange(n, dtype=np.uint32))
    ab = spec["a_plus_b"]
    pk = ab ** (s - np.arange(s + 1)) * (1 - ab) ** np.arange(s + 1)
    deg = np.rint(m * pk[k]).astype(np.uint64)
    rp = np.zeros(n + 1, dtype=np.uint64)
    np.cumsum(deg, out=rp[1:])
    del deg, k
    plan = G.gts_plan_pages(rp, page_bytes=1 << 20)
    total = plan["num_pages"]
    assert abs(total - spec["paper_total_pages"]) <= spec["rel_tol_total"] * spec["paper_total_pages"], plan
    assert abs(plan["n_lp"] - spec["paper_lp_pages"]) <= spec["lp_abs_tol"], plan


def test_rejects_bad_input():
    g = inputs.path(5)
    with pytest.raises(G.GtsError) as e:
        G.gts_build_pages(g.row_ptr, np.array([0, 1, 2, 9], dtype=np.uint32))
    assert e.value.code == G.GTS_EINVAL
    with pytest.raises(G.GtsError):
        G.gts_build_pages(g.row_ptr, g.col, page_bytes=3000)
    bad = g.row_ptr.copy()
    bad[2], bad[3] = bad[3], bad[2]
    with pytest.raises(G.GtsError):
        G.gts_build_pages(bad, g.col)
    with pytest.raises(G.GtsError) as e:        # PID16: > 65536 slots is fine, > 65536 pages is not
        G.gts_build_pages(*[inputs.from_edges(1_400_000, []).row_ptr, np.zeros(0, np.uint32)], page_bytes=256,
                          entry_encoding=G.GTS_ENTRY_PID16_SLOT16)
    assert e.value.code == G.GTS_EOVERFLOW


def test_hot_table_holds_top_in_degree():
    g = inputs.rmat(16)
    gr = G.gts_build_pages(g.row_ptr, g.col)
    st = gr.stats()
    indeg = np.bincount(g.col, minlength=g.n)
    # at least the 1,000 hottest vertices have in-degree >= 64 and must all be in the table
    assert st["n_hot"] >= 1000


def test_degree_order_build():
    """GTS_BUILD_DEGREE_ORDER: pages hold the graph renamed by descending in-degree."""
    g = inputs.rmat(13).with_weights()
    gr = G.gts_build_pages(g.row_ptr, g.col, g.weights, page_bytes=8192, order=True)
    st = gr.stats()
    assert st["ordered"] == 1
    p = gr.order()
    assert np.array_equal(np.sort(p), np.arange(g.n))
    indeg = np.bincount(g.col, minlength=g.n)
    assert np.all(np.diff(indeg[np.argsort(p)]) <= 0)           # internal order = descending in-degree
    assert np.array_equal(p, inputs.indegree_order(g))
    h = inputs.permute(g, p)
    rp, col, w = oracle.decode_pages(gr.pages(), 8192, g.n, g.m, weighted=True)
    assert np.array_equal(rp, h.row_ptr) and np.array_equal(col, h.col)
    # weights travel with their edges: compare (src, dst, w) multisets
    src = np.repeat(np.arange(g.n), np.diff(g.row_ptr).astype(np.int64))
    a = sorted(zip(p[src].tolist(), p[g.col].tolist(), g.weights.tolist()))
    src2 = np.repeat(np.arange(g.n), np.diff(rp).astype(np.int64))
    b = sorted(zip(src2.tolist(), col.tolist(), w.tolist()))
    assert a == b
    plain = G.gts_build_pages(g.row_ptr, g.col, page_bytes=8192)
    assert np.array_equal(plain.order(), np.arange(g.n))


def _symmetrised(g):
    """CSR of the multigraph with every edge u->v also stored as v->u (rows sorted)."""
    src = np.repeat(np.arange(g.n), np.diff(g.row_ptr).astype(np.int64))
    s = np.concatenate([src, g.col.astype(np.int64)])
    d = np.concatenate([g.col.astype(np.int64), src])
    order = np.lexsort((d, s))
    rp = np.zeros(g.n + 1, np.uint64)
    rp[1:] = np.cumsum(np.bincount(s, minlength=g.n))
    return rp, d[order].astype(np.uint32)


@pytest.mark.parametrize("maker", [lambda: inputs.rmat(12), lambda: inputs.random_graph(3000, 9000, 5),
                                   lambda: inputs.in_star(5000)])
@pytest.mark.parametrize("order", [False, True])
def test_symmetric_build_round_trip(maker, order):
    """GTS_BUILD_SYMMETRIC (SURVEY 8(e) WCC caveat): the pages hold every edge in both
    directions; the oracle's independent page reader recovers exactly the symmetrised
    CSR (in internal IDs for degree-ordered pages)."""
    g = maker()
    gr = G.gts_build_pages(g.row_ptr, g.col, page_bytes=4096, symmetric=True, order=order)
    st = gr.stats()
    assert st["symmetric"] == 1 and st["m"] == 2 * g.m
    rp, col = _symmetrised(g)
    if order:
        new = gr.order()
        perm = inputs.permute(inputs.CSR(rp, col), new)
        rp, col = perm.row_ptr, perm.col
    drp, dcol, _ = oracle.decode_pages(gr.pages(), 4096, g.n, 2 * g.m)
    assert np.array_equal(drp, rp)
    assert np.array_equal(dcol, col)


@pytest.mark.parametrize("strategy", [0, 1, 2])
@pytest.mark.parametrize("world", [2, 3, 8])
def test_owner_filtered_builds_partition_the_pages(strategy, world):
    """GTS_BUILD_OWNER_FILTER: rank r of an N-rank job builds and holds only the pages it
    processes (P: j mod N; S: its contiguous range; S_BCAST: all).
    The held pages are byte-identical to the full build's, the ranks' page sets
    partition the graph (P, S), and the host bytes per rank are ~T_topo / N."""
    g = inputs.rmat(13)
    pb = 4096
    full = G.gts_build_pages(g.row_ptr, g.col, page_bytes=pb, order=True)
    fp = full.pages().reshape(-1, pb)
    P = fp.shape[0]
    owner, _ = G.gts_partition_pages(full, strategy, world)
    seen = np.zeros(P, np.int64)
    tot = 0
    for r in range(world):
        gr = G.gts_build_pages(g.row_ptr, g.col, page_bytes=pb, order=True, owner=(r, world, strategy))
        st = gr.stats()
        assert st["owner_rank"] == r and st["owner_world"] == world
        mine = np.arange(P) if strategy == 2 else np.nonzero(owner == r)[0]
        assert st["host_page_bytes"] == len(mine) * pb
        assert np.array_equal(gr.pages().reshape(-1, pb), fp[mine])
        assert np.array_equal(gr.directory()["start_vid"], full.directory()["start_vid"])
        seen[mine] += 1
        tot += st["host_page_bytes"]
    if strategy != 2:
        assert np.all(seen == 1) and tot == P * pb
        assert max(np.bincount(owner, minlength=world)) <= -(-P // world) + 1 + 2   # ~T_topo / N per rank


def test_owner_filter_rejects_bad_rank():
    g = inputs.rmat(10)
    with pytest.raises(G.GtsError) as e:
        G.gts_build_pages(g.row_ptr, g.col, page_bytes=4096, owner=(3, 3, 0))
    assert e.value.code == G.GTS_EINVAL
