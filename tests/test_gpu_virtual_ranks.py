"""Every multi-GPU merge path of libgts, run on one GPU.

gts_run_config.virtual_ranks = V runs the V-rank job of a strategy on this
GPU: each rank's page set, WA buffers, sweep kernels, merge kernels, route
packing / capacity exchange / apply run as on V GPUs; only the transport of
the collectives is device memory instead of NCCL.

For V in {2, 3, 8}, every strategy (P: pages h(j) = j mod N, WA replicated,
P:344-354; S: WA range-partitioned with routed updates, P:430-440 + north_star;
S_BCAST: the paper-literal S) and every algorithm, the result must equal the
oracle: bit-exact for BFS / SSSP / WCC, PageRank within max rel 1e-4 and L1
1e-5.  WCC under S runs routed label propagation on GTS_BUILD_SYMMETRIC pages.
"""
import numpy as np
import pytest

import inputs
import oracle

pytestmark = pytest.mark.gpu

STRATS = {"P": 0, "S": 1, "SB": 2}
VS = [2, 3, 8]


@pytest.fixture(scope="module")
def G():
    import paper_conf_sigmod_0002apsk16_b200 as G
    return G


@pytest.fixture(scope="module")
def ctx(G, gpu):
    c = G.gts_context_create(0)
    yield c
    c.free()


_cache = {}


def case(name):
    if name not in _cache:
        if name == "rmat16_4k":
            g, pb = inputs.rmat(16), 4096
        elif name == "twitter16":
            g, pb = inputs.twitter_like(n=1 << 16, m=1 << 20), 8192
        elif name == "instar":
            g, pb = inputs.in_star(100000), 4096
        elif name == "rand":
            g, pb = inputs.random_graph(30000, 150000, 7), 4096
        else:
            raise KeyError(name)
        _cache[name] = (g, pb)
    return _cache[name]


GRAPHS = ["rmat16_4k", "twitter16", "rand"]


def pr_ok(got, want):
    rel = np.abs(got.astype(np.float64) - want) / want
    return rel.max() <= 1e-4 and np.abs(got - want).sum() <= 1e-5, float(rel.max())


@pytest.mark.parametrize("name", GRAPHS)
@pytest.mark.parametrize("order", [False, True])
@pytest.mark.parametrize("strat", list(STRATS))
@pytest.mark.parametrize("V", VS)
def test_bfs(G, ctx, name, order, strat, V):
    g, pb = case(name)
    gr = G.gts_build_pages(g.row_ptr, g.col, page_bytes=pb, order=order)
    deg = np.diff(g.row_ptr)
    for src in (0, int(np.argmax(deg)), g.n - 1):
        want = oracle.bfs(g.row_ptr, g.col, src)
        got, st = G.gts_bfs(ctx, gr, src, strategy=STRATS[strat], virtual_ranks=V)
        assert np.array_equal(got, want), (name, strat, V, src, int(np.sum(got != want)))
        assert st["edges_traversed"] == int(deg[want != oracle.UNREACHED].astype(np.int64).sum()) or strat == "SB"
        if strat == "S" and V > 1:
            assert st["routed_msgs"] > 0 or st["levels_or_iters"] <= 2


@pytest.mark.parametrize("name", GRAPHS)
@pytest.mark.parametrize("strat", list(STRATS))
@pytest.mark.parametrize("V", VS)
def test_sssp(G, ctx, name, strat, V):
    g, pb = case(name)
    w = inputs.edge_weights(g)
    gr = G.gts_build_pages(g.row_ptr, g.col, w, page_bytes=pb, order=(V == 3))
    for src in (0, int(np.argmax(np.diff(g.row_ptr)))):
        want = oracle.sssp(g.row_ptr, g.col, w, src)
        got, _ = G.gts_sssp(ctx, gr, src, strategy=STRATS[strat], virtual_ranks=V)
        assert np.array_equal(got, want), (name, strat, V, src, int(np.sum(got != want)))
    # near-far buckets on the multi-rank path (any delta gives the exact distances)
    got, _ = G.gts_sssp(ctx, gr, 0, strategy=STRATS[strat], virtual_ranks=V, tune={"sssp_delta": 64})
    assert np.array_equal(got, oracle.sssp(g.row_ptr, g.col, w, 0))


@pytest.mark.parametrize("name", GRAPHS + ["instar"])
@pytest.mark.parametrize("order", [False, True])
@pytest.mark.parametrize("strat", list(STRATS))
@pytest.mark.parametrize("V", VS)
def test_pagerank(G, ctx, name, order, strat, V):
    g, pb = case(name)
    gr = G.gts_build_pages(g.row_ptr, g.col, page_bytes=pb, order=order)
    for dangling in (0, 1):
        want = oracle.pagerank(g.row_ptr, g.col, 10, 0.85, dangling=dangling)
        got, st = G.gts_pagerank(ctx, gr, 10, 0.85, dangling=dangling, strategy=STRATS[strat], virtual_ranks=V)
        ok, rel = pr_ok(got, want)
        assert ok, (name, order, strat, V, dangling, rel)


@pytest.mark.parametrize("name", GRAPHS)
@pytest.mark.parametrize("order", [False, True])
@pytest.mark.parametrize("strat", list(STRATS))
@pytest.mark.parametrize("V", VS)
def test_wcc(G, ctx, name, order, strat, V):
    g, pb = case(name)
    want = oracle.wcc(g.row_ptr, g.col)
    # Strategy-S pushes labels along both directions from the source's owner: symmetrised pages
    gr = G.gts_build_pages(g.row_ptr, g.col, page_bytes=pb, order=order, symmetric=(strat == "S"))
    got, st = G.gts_wcc(ctx, gr, strategy=STRATS[strat], virtual_ranks=V)
    assert np.array_equal(got, want), (name, order, strat, V, int(np.sum(got != want)))


def test_wcc_strategy_s_needs_symmetric_pages(G, ctx):
    g, pb = case("rand")
    gr = G.gts_build_pages(g.row_ptr, g.col, page_bytes=pb)
    with pytest.raises(G.GtsError) as e:
        G.gts_wcc(ctx, gr, strategy=STRATS["S"], virtual_ranks=2)
    assert e.value.code == G.GTS_EUNSUPPORTED


@pytest.mark.parametrize("strat", list(STRATS))
def test_streamed_virtual_ranks(G, ctx, strat):
    """Pages streamed from pinned host memory through the ring, per virtual rank."""
    g, pb = case("rmat16_4k")
    w = inputs.edge_weights(g)
    gr = G.gts_build_pages(g.row_ptr, g.col, page_bytes=pb, order=True)
    grw = G.gts_build_pages(g.row_ptr, g.col, w, page_bytes=pb)
    grs = G.gts_build_pages(g.row_ptr, g.col, page_bytes=pb, symmetric=True)
    kw = dict(strategy=STRATS[strat], virtual_ranks=3, residency=G.GTS_STREAMED, batch_pages=8, ring_slots=2)
    got, st = G.gts_bfs(ctx, gr, 0, **kw)
    assert np.array_equal(got, oracle.bfs(g.row_ptr, g.col, 0))
    assert st["h2d_bytes"] > 0
    got, _ = G.gts_sssp(ctx, grw, 0, **kw)
    assert np.array_equal(got, oracle.sssp(g.row_ptr, g.col, w, 0))
    got, _ = G.gts_pagerank(ctx, gr, 10, 0.85, **kw)
    assert pr_ok(got, oracle.pagerank(g.row_ptr, g.col, 10, 0.85))[0]
    got, _ = G.gts_wcc(ctx, grs if strat == "S" else gr, **kw)
    assert np.array_equal(got, oracle.wcc(g.row_ptr, g.col))


@pytest.mark.parametrize("V", [2, 4, 8])
def test_strategy_s_wa_per_rank(G, ctx, V):
    """Strategy-S: each rank allocates its WA range only (logically one GPU of
    large memory), so the per-rank attribute bytes shrink with N; Strategy-P replicates them."""
    g, pb = case("rmat16_4k")
    gr = G.gts_build_pages(g.row_ptr, g.col, page_bytes=pb)
    n = g.n
    _, sp = G.gts_pagerank(ctx, gr, 2, 0.85, strategy=0, virtual_ranks=V)
    _, ss = G.gts_pagerank(ctx, gr, 2, 0.85, strategy=1, virtual_ranks=V)
    assert sp["wa_bytes"] == 8 * n
    # x + acc over rank 0's range (~n/V) + the dense hot partials
    assert ss["wa_bytes"] <= 8 * n / V * 1.5 + 4 * min(n, 53248)
    _, bp = G.gts_bfs(ctx, gr, 0, strategy=0, virtual_ranks=V)
    _, bs = G.gts_bfs(ctx, gr, 0, strategy=1, virtual_ranks=V)
    assert bs["wa_bytes"] < bp["wa_bytes"]
    assert bs["wa_bytes"] <= (4 * n + 12 * n / 32) / V * 1.5 + n / 8 + 64


def test_virtual_ranks_rejected_on_bad_values(G, ctx):
    g, pb = case("rand")
    gr = G.gts_build_pages(g.row_ptr, g.col, page_bytes=pb)
    with pytest.raises(G.GtsError):
        G.gts_bfs(ctx, gr, 0, virtual_ranks=9)
    with pytest.raises(G.GtsError) as e:
        G.gts_bfs(ctx, gr, 0, virtual_ranks=2, micro="edge")
    assert e.value.code == G.GTS_EUNSUPPORTED


@pytest.mark.parametrize("name", GRAPHS + ["instar"])
@pytest.mark.parametrize("order", [False, True])
@pytest.mark.parametrize("V", VS)
def test_pagerank_strategy_s_peer(G, ctx, name, order, V):
    """GTS_ROUTE_PEER: the Strategy-S scatter adds every remote update (and every remote
    hot partial) straight into the owner's WA -- the fused scatter + exchange over peer
    memory -- with WA double-buffered across iterations; same result as the oracle."""
    g, pb = case(name)
    gr = G.gts_build_pages(g.row_ptr, g.col, page_bytes=pb, order=order)
    for dangling in (0, 1):
        want = oracle.pagerank(g.row_ptr, g.col, 10, 0.85, dangling=dangling)
        got, st = G.gts_pagerank(ctx, gr, 10, 0.85, dangling=dangling, strategy=STRATS["S"], virtual_ranks=V,
                                 route_peer=True)
        ok, rel = pr_ok(got, want)
        assert ok, (name, order, V, dangling, rel)
        assert st["routed_msgs"] == 0
    got, _ = G.gts_pagerank(ctx, gr, 10, 0.85, strategy=STRATS["S"], virtual_ranks=V, route_peer=True,
                            residency=G.GTS_STREAMED, batch_pages=4, ring_slots=2)
    assert pr_ok(got, oracle.pagerank(g.row_ptr, g.col, 10, 0.85))[0]


@pytest.mark.parametrize("name", GRAPHS)
@pytest.mark.parametrize("V", VS)
def test_bfs_sssp_wcc_strategy_s_peer(G, ctx, name, V):
    """GTS_ROUTE_PEER for the BFS-like algorithms: remote discoveries / relaxations / label
    updates are atomics in the owner's visited / next bitmaps, dist and labels (the next
    bitmaps alternate by level); bit-exact vs the oracle, resident and streamed."""
    g, pb = case(name)
    w = inputs.edge_weights(g)
    gr = G.gts_build_pages(g.row_ptr, g.col, page_bytes=pb, order=True)
    grw = G.gts_build_pages(g.row_ptr, g.col, w, page_bytes=pb)
    grs = G.gts_build_pages(g.row_ptr, g.col, page_bytes=pb, symmetric=True, order=(V == 3))
    for kw in ({}, dict(residency=G.GTS_STREAMED, batch_pages=4, ring_slots=2)):
        kw = dict(kw, strategy=STRATS["S"], virtual_ranks=V, route_peer=True)
        for src in (0, int(np.argmax(np.diff(g.row_ptr)))):
            got, st = G.gts_bfs(ctx, gr, src, **kw)
            assert np.array_equal(got, oracle.bfs(g.row_ptr, g.col, src)), (name, V, src, kw)
            assert st["routed_msgs"] == 0
            got, _ = G.gts_sssp(ctx, grw, src, **kw)
            assert np.array_equal(got, oracle.sssp(g.row_ptr, g.col, w, src)), (name, V, src, kw)
        got, _ = G.gts_wcc(ctx, grs, **kw)
        assert np.array_equal(got, oracle.wcc(g.row_ptr, g.col)), (name, V, kw)
    got, _ = G.gts_sssp(ctx, grw, 0, strategy=STRATS["S"], virtual_ranks=V, route_peer=True, tune={"sssp_delta": 32})
    assert np.array_equal(got, oracle.sssp(g.row_ptr, g.col, w, 0))
