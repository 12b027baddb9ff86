"""Pins for oracle.sssp (BFS-like class P:308, App D; R11) and
oracle.wcc ("connected components"; R12).

SSSP: Bellman-Ford brute force on tiny graphs, unit weights == BFS, weighted
path prefix sums, scipy dijkstra (min over parallel edges), feasibility and
tightness invariants.  WCC: scipy connected_components(weak) partitions,
closed forms, invariants.
"""
import numpy as np
import pytest
import scipy.sparse as sp
from scipy.sparse import csgraph

import inputs
import oracle

U = oracle.UNREACHED


def bellman_ford(n, edges, w, src):
    INF = float("inf")
    d = [INF] * n
    d[src] = 0
    for _ in range(n):
        for (u, v), c in zip(edges, w):
            if d[u] + c < d[v]:
                d[v] = d[u] + c
    return [U if x == INF else int(x) for x in d]


def test_sssp_bellman_ford_small():
    rng = np.random.default_rng(3)
    for _ in range(300):
        n = int(rng.integers(1, 10))
        m = int(rng.integers(0, 4 * n + 1))
        edges = rng.integers(0, n, size=(m, 2)).tolist()
        w = rng.integers(1, 256, size=m).tolist()
        g = inputs.from_edges(n, edges, w)
        src = int(rng.integers(0, n))
        assert oracle.sssp(g.row_ptr, g.col, g.weights, src).tolist() == bellman_ford(n, edges, w, src)


def test_sssp_unit_weights_equal_bfs():
    g = inputs.rmat(13)
    w = np.ones(g.m, dtype=np.uint32)
    for src in (0, 3):
        assert np.array_equal(oracle.sssp(g.row_ptr, g.col, w, src), oracle.bfs(g.row_ptr, g.col, src))


def test_sssp_weighted_path_prefix_sums():
    n = 500
    rng = np.random.default_rng(5)
    w = rng.integers(1, 256, size=n - 1)
    g = inputs.from_edges(n, [(i, i + 1) for i in range(n - 1)], w)
    d = oracle.sssp(g.row_ptr, g.col, g.weights, 0)
    assert np.array_equal(d, np.concatenate([[0], np.cumsum(w)]).astype(np.uint32))


def _scipy_dist(g, src):
    src_of = np.repeat(np.arange(g.n), np.diff(g.row_ptr).astype(np.int64))
    # parallel edges: keep the minimum weight (csr_matrix would sum duplicates)
    order = np.lexsort((g.weights, g.col, src_of))
    s, t, w = src_of[order], g.col[order].astype(np.int64), g.weights[order].astype(np.float64)
    first = np.ones(len(s), dtype=bool)
    first[1:] = (s[1:] != s[:-1]) | (t[1:] != t[:-1])
    A = sp.csr_matrix((w[first], (s[first], t[first])), shape=(g.n, g.n))
    d = csgraph.dijkstra(A, directed=True, indices=src)
    return np.where(np.isinf(d), U, d).astype(np.uint32)


@pytest.mark.parametrize("scale", [10, 14])
def test_sssp_vs_scipy_rmat(scale):
    g = inputs.rmat(scale).with_weights()
    for src in (0, 2):
        assert np.array_equal(oracle.sssp(g.row_ptr, g.col, g.weights, src), _scipy_dist(g, src))


def test_sssp_invariants():
    g = inputs.rmat(14).with_weights()
    d = oracle.sssp(g.row_ptr, g.col, g.weights, 0).astype(np.int64)
    src_of = np.repeat(np.arange(g.n), np.diff(g.row_ptr).astype(np.int64))
    t = g.col.astype(np.int64)
    w = g.weights.astype(np.int64)
    r = d[src_of] != U
    assert np.all(d[t[r]] <= d[src_of[r]] + w[r])          # feasible
    tight = np.zeros(g.n, dtype=bool)
    tight[t[r & (d[t] == d[src_of] + w)]] = True
    reached = d != U
    reached[0] = False
    assert np.all(tight[reached])                            # every reached v has a tight in-edge


def test_sssp_overflow_detected():
    g = inputs.from_edges(3, [(0, 1), (1, 2)], [0xFFFFFFF0, 0x20])
    with pytest.raises(OverflowError):
        oracle.sssp(g.row_ptr, g.col, g.weights, 0)


# ------------------------------------------------------------------ WCC ---

def _scipy_labels(g):
    A = sp.csr_matrix((np.ones(g.m), g.col.astype(np.int64), g.row_ptr.astype(np.int64)), shape=(g.n, g.n))
    k, comp = csgraph.connected_components(A, directed=True, connection="weak")
    minv = np.full(k, np.iinfo(np.int64).max)
    np.minimum.at(minv, comp, np.arange(g.n))
    return minv[comp].astype(np.uint32)


@pytest.mark.parametrize("maker", [lambda: inputs.rmat(12), lambda: inputs.rmat(16),
                                   lambda: inputs.random_graph(5000, 4000, 1),
                                   lambda: inputs.twitter_like(n=30000, m=90000)])
def test_wcc_vs_scipy(maker):
    g = maker()
    assert np.array_equal(oracle.wcc(g.row_ptr, g.col), _scipy_labels(g))


def test_wcc_closed_forms():
    k, L = 7, 13
    edges = [(c * L + i, c * L + (i + 1) % L) for c in range(k) for i in range(L)]
    g = inputs.from_edges(k * L, edges)
    lab = oracle.wcc(g.row_ptr, g.col)
    assert len(np.unique(lab)) == k
    assert np.array_equal(lab, (np.arange(k * L) // L) * L)
    g = inputs.path(100)
    assert np.all(oracle.wcc(g.row_ptr, g.col) == 0)
    g = inputs.from_edges(10, [])
    assert np.array_equal(oracle.wcc(g.row_ptr, g.col), np.arange(10))
    # direction is ignored: in-star hub 5 of leaves > 5 and < 5
    g = inputs.from_edges(9, [(v, 5) for v in range(9) if v != 5])
    assert np.all(oracle.wcc(g.row_ptr, g.col) == 0)


def test_wcc_invariants():
    g = inputs.rmat(15)
    lab = oracle.wcc(g.row_ptr, g.col).astype(np.int64)
    src_of = np.repeat(np.arange(g.n), np.diff(g.row_ptr).astype(np.int64))
    assert np.all(lab[src_of] == lab[g.col.astype(np.int64)])
    assert np.all(lab <= np.arange(g.n))
    assert np.array_equal(lab[lab], lab)
