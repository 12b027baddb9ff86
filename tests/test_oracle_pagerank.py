"""Pins for oracle.pagerank (Alg 4/5 P:1540-1558, P:1528-1532, P:338;
readings R1-R5 in DESIGN.md).

Checked against closed forms (cycle, edgeless, complete digraph, in-star
two-variable recurrence), a dense-matrix power iteration in numpy, networkx at
convergence, and invariants (sum = 1 in UNIFORM mode; the DROP-mode mass
identity; x_v >= (1-d)/n).
"""
import networkx as nx
import numpy as np
import pytest

import inputs
import oracle

D = 0.85


def test_cycle_is_uniform():
    for n in (1, 2, 7, 1000):
        g = inputs.cycle(n)
        x = oracle.pagerank(g.row_ptr, g.col, 10, D)
        assert np.allclose(x, 1.0 / n, rtol=1e-14, atol=0)


def test_edgeless_uniform_and_drop():
    n = 50
    g = inputs.from_edges(n, [])
    x = oracle.pagerank(g.row_ptr, g.col, 10, D)
    assert np.allclose(x, 1.0 / n, rtol=1e-14, atol=0)
    # paper-literal (dangling mass dropped): after one iteration x = (1-d)/n
    x = oracle.pagerank(g.row_ptr, g.col, 1, D, dangling=oracle.DANGLING_DROP)
    assert np.allclose(x, (1 - D) / n, rtol=1e-14, atol=0)


def test_complete_digraph_is_uniform():
    n = 30
    g = inputs.from_edges(n, [(u, v) for u in range(n) for v in range(n) if u != v])
    x = oracle.pagerank(g.row_ptr, g.col, 10, D)
    assert np.allclose(x, 1.0 / n, rtol=1e-13, atol=0)


def _instar_closed_form(k, iters, d):
    """In-star: k leaves -> hub, hub dangling, n = k+1 (SURVEY.md 8(c) hub pin).
    l^t = (1-d)/n + d*eta/n ;  eta^t = (1-d)/n + d*(k*l/1 + eta/n)  (leaf outdeg 1)."""
    n = k + 1
    leaf = eta = 1.0 / n
    for _ in range(iters):
        leaf, eta = (1 - d) / n + d * eta / n, (1 - d) / n + d * (k * leaf + eta / n)
    return leaf, eta


@pytest.mark.parametrize("k", [1, 5, 1000, 100_000])
def test_in_star_closed_form(k):
    g = inputs.in_star(k)
    x = oracle.pagerank(g.row_ptr, g.col, 10, D)
    leaf, eta = _instar_closed_form(k, 10, D)
    # the oracle sums k fp64 terms sequentially: |err| <= (k-1) * 2^-53 * sum (Higham 4.2)
    assert abs(x[0] - eta) <= (1e-14 + k * 2.0 ** -53) * eta
    assert np.allclose(x[1:], leaf, rtol=1e-14 + k * 2.0 ** -53, atol=0)


def _dense_pagerank(g, iters, d, uniform=True):
    n = g.n
    A = np.zeros((n, n))
    src = np.repeat(np.arange(n), np.diff(g.row_ptr).astype(np.int64))
    np.add.at(A, (g.col.astype(np.int64), src), 1.0)  # A[v,u] = multiplicity of u->v
    deg = np.diff(g.row_ptr).astype(np.float64)
    P = np.where(deg > 0, A / np.where(deg > 0, deg, 1.0), 0.0)
    if uniform:
        P = P + np.where(deg == 0, 1.0 / n, 0.0)[None, :]
    G = d * P + (1 - d) / n * (np.ones((n, n)) if uniform else 0.0)
    x = np.full(n, 1.0 / n)
    if uniform:
        return np.linalg.matrix_power(G, iters) @ x
    for _ in range(iters):
        x = d * P @ x + (1 - d) / n
    return x


@pytest.mark.parametrize("seed", range(6))
def test_dense_matrix_power(seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(2, 300))
    g = inputs.random_graph(n, int(rng.integers(0, 4 * n)), seed)
    for uniform in (True, False):
        mode = oracle.DANGLING_UNIFORM if uniform else oracle.DANGLING_DROP
        x = oracle.pagerank(g.row_ptr, g.col, 10, D, dangling=mode)
        ref = _dense_pagerank(g, 10, D, uniform)
        assert np.max(np.abs(x - ref)) <= 1e-13


def test_networkx_at_convergence():
    g = inputs.random_graph(200, 700, 7, self_loops=False)
    src = np.repeat(np.arange(g.n), np.diff(g.row_ptr).astype(np.int64))
    G = nx.DiGraph()
    G.add_nodes_from(range(g.n))
    pairs = set(zip(src.tolist(), g.col.tolist()))
    if len(pairs) != g.m:      # keep it a simple digraph
        g = inputs.from_edges(g.n, sorted(pairs))
    G.add_edges_from(pairs)
    ref = nx.pagerank(G, alpha=D, tol=1e-15, max_iter=2000)
    x = oracle.pagerank(g.row_ptr, g.col, 200, D)
    assert max(abs(x[v] - ref[v]) for v in range(g.n)) <= 1e-12


def test_invariants_rmat():
    g = inputs.rmat(14)
    x = oracle.pagerank(g.row_ptr, g.col, 10, D)
    assert abs(np.sum(np.sort(x)) - 1.0) <= 1e-9
    assert np.all(x >= (1 - D) / g.n * (1 - 1e-12))
    # DROP: sum x^t = (1-d) + d * sum_{u: outdeg>0} x_u^{t-1}
    deg = np.diff(g.row_ptr)
    x9 = oracle.pagerank(g.row_ptr, g.col, 9, D, dangling=oracle.DANGLING_DROP)
    x10 = oracle.pagerank(g.row_ptr, g.col, 10, D, dangling=oracle.DANGLING_DROP)
    assert abs(x10.sum() - ((1 - D) + D * x9[deg > 0].sum())) <= 1e-12
    assert x10.sum() < 1.0


def test_two_vertex_recurrence():
    g = inputs.from_edges(2, [(0, 1)])
    x = oracle.pagerank(g.row_ptr, g.col, 10, D)
    u = v = 0.5
    for _ in range(10):   # D = v (vertex 1 dangling)
        u, v = (1 - D) / 2 + D * v / 2, (1 - D) / 2 + D * (u + v / 2)
    assert abs(x[0] - u) < 1e-15 and abs(x[1] - v) < 1e-15


def test_multiedges_count_with_multiplicity():
    g = inputs.from_edges(3, [(0, 1), (0, 1), (0, 2), (1, 0), (2, 0)])
    x = oracle.pagerank(g.row_ptr, g.col, 10, D)
    assert np.max(np.abs(x - _dense_pagerank(g, 10, D))) < 1e-15


@pytest.mark.parametrize("maker", [lambda: inputs.rmat(16), lambda: inputs.random_graph(30000, 200000, 5),
                                   lambda: inputs.in_star(100000)])
@pytest.mark.parametrize("dangling", [oracle.DANGLING_UNIFORM, oracle.DANGLING_DROP])
def test_openmp_build_byte_identical(maker, dangling):
    """the oracle is compiled plain and with OpenMP; every y[v]
    sums its in-edges in ascending u in both builds and D is summed
    sequentially, so the outputs are byte-identical (the OpenMP build is the
    parity reference at full size and the all-core CPU baseline)."""
    g = maker()
    a = oracle.pagerank(g.row_ptr, g.col, 10, D, dangling=dangling, omp=False)
    b = oracle.pagerank(g.row_ptr, g.col, 10, D, dangling=dangling, omp=True)
    assert a.tobytes() == b.tobytes()
    assert oracle.num_threads(omp=False) == 1
