"""Pins for oracle.bfs (Alg 2/3; out-edges P:538).

The oracle is a FIFO-queue BFS.  It is checked here against things that are not
itself: a brute-force relaxation fixpoint (a different algorithm) on every
digraph with n <= 3 (self-loops included) and every loop-free digraph with
n = 4, closed forms, scipy.sparse.csgraph and invariants.
"""
import itertools

import numpy as np
import pytest
import scipy.sparse as sp
from scipy.sparse import csgraph

import inputs
import oracle

U = oracle.UNREACHED


def brute_levels(n, edges, src):
    """Repeated relaxation until fixpoint: L[v] = min over u->v of L[u]+1."""
    INF = float("inf")
    L = [INF] * n
    L[src] = 0
    changed = True
    while changed:
        changed = False
        for u, v in edges:
            if L[u] + 1 < L[v]:
                L[v] = L[u] + 1
                changed = True
    return [U if x == INF else int(x) for x in L]


def _all_digraphs(n, self_loops):
    pairs = [(u, v) for u in range(n) for v in range(n) if self_loops or u != v]
    for mask in range(1 << len(pairs)):
        yield [pairs[i] for i in range(len(pairs)) if mask >> i & 1]


@pytest.mark.parametrize("n,self_loops", [(1, True), (2, True), (3, True), (4, False)])
def test_bfs_all_small_digraphs(n, self_loops):
    for edges in _all_digraphs(n, self_loops):
        g = inputs.from_edges(n, edges)
        for src in range(n):
            got = oracle.bfs(g.row_ptr, g.col, src).tolist()
            assert got == brute_levels(n, edges, src), (edges, src)


def test_bfs_random_small_multigraphs():
    rng = np.random.default_rng(1)
    for t in range(400):
        n = int(rng.integers(1, 13))
        m = int(rng.integers(0, 3 * n + 1))
        edges = rng.integers(0, n, size=(m, 2)).tolist()
        g = inputs.from_edges(n, edges)
        src = int(rng.integers(0, n))
        assert oracle.bfs(g.row_ptr, g.col, src).tolist() == brute_levels(n, edges, src)


def test_bfs_closed_forms():
    n = 1000
    g = inputs.path(n)
    assert np.array_equal(oracle.bfs(g.row_ptr, g.col, 0), np.arange(n, dtype=np.uint32))
    lv = oracle.bfs(g.row_ptr, g.col, 10)
    assert np.all(lv[:10] == U) and np.array_equal(lv[10:], np.arange(n - 10))
    g = inputs.cycle(n)
    s = 123
    assert np.array_equal(oracle.bfs(g.row_ptr, g.col, s), (np.arange(n) - s) % n)
    g = inputs.out_star(500)
    lv = oracle.bfs(g.row_ptr, g.col, 0)
    assert lv[0] == 0 and np.all(lv[1:] == 1)
    g = inputs.in_star(500)
    lv = oracle.bfs(g.row_ptr, g.col, 0)
    assert lv[0] == 0 and np.all(lv[1:] == U)
    lv = oracle.bfs(g.row_ptr, g.col, 7)
    assert lv[7] == 0 and lv[0] == 1 and (lv == U).sum() == 499
    g = inputs.binary_tree(4095)
    v = np.arange(4095)
    assert np.array_equal(oracle.bfs(g.row_ptr, g.col, 0), np.floor(np.log2(v + 1)).astype(np.uint32))


def _scipy_levels(g, src):
    A = sp.csr_matrix((np.ones(g.m), g.col.astype(np.int64), g.row_ptr.astype(np.int64)), shape=(g.n, g.n))
    d = csgraph.shortest_path(A, method="D", directed=True, unweighted=True, indices=src)
    return np.where(np.isinf(d), U, d).astype(np.uint32)


@pytest.mark.parametrize("scale", [10, 13])
def test_bfs_vs_scipy_rmat(scale):
    g = inputs.rmat(scale)
    for src in (0, 1, 5, g.n - 1):
        assert np.array_equal(oracle.bfs(g.row_ptr, g.col, src), _scipy_levels(g, src))


def test_bfs_vs_scipy_twitter_like():
    g = inputs.twitter_like(n=20000, m=200000)
    for src in (0, 17):
        assert np.array_equal(oracle.bfs(g.row_ptr, g.col, src), _scipy_levels(g, src))


def test_bfs_invariants_rmat16():
    g = inputs.rmat(16)
    lv = oracle.bfs(g.row_ptr, g.col, 0).astype(np.int64)
    src_of = np.repeat(np.arange(g.n), np.diff(g.row_ptr).astype(np.int64))
    dst = g.col.astype(np.int64)
    reached_u = lv[src_of] != U
    # every edge u->v with u reached: level v <= level u + 1 (and v reached)
    assert np.all(lv[dst[reached_u]] != U)
    assert np.all(lv[dst[reached_u]] <= lv[src_of[reached_u]] + 1)
    # every reached v != src has an in-neighbour at level v - 1
    tight = np.zeros(g.n, dtype=bool)
    ok = reached_u & (lv[dst] == lv[src_of] + 1)
    tight[dst[ok]] = True
    reached = lv != U
    reached[0] = False
    assert np.all(tight[reached])
    # survey's RMAT-20 shape check at 16: BFS from 0 reaches most edges
    deg = np.diff(g.row_ptr).astype(np.int64)
    assert deg[lv != U].sum() > 0.95 * g.m


def test_bfs_symmetrised_abs_difference():
    """North_star invariant: |level(u) - level(v)| <= 1 across every undirected edge."""
    g = inputs.rmat(12)
    src_of = np.repeat(np.arange(g.n), np.diff(g.row_ptr).astype(np.int64))
    e = np.concatenate([np.stack([src_of, g.col], 1), np.stack([g.col, src_of], 1)])
    s = inputs.from_edges(g.n, e)
    lv = oracle.bfs(s.row_ptr, s.col, 0).astype(np.int64)
    a, b = lv[e[:, 0]], lv[e[:, 1]]
    both = (a != U) & (b != U)
    assert np.all(np.abs(a[both] - b[both]) <= 1)
    assert np.all((a == U) == (b == U))


def test_bfs_rejects_bad_src():
    g = inputs.path(3)
    with pytest.raises(ValueError):
        oracle.bfs(g.row_ptr, g.col, 3)


def test_generator_lean_mode_same_graph():
    a = inputs.rmat(13)
    b = inputs.rmat(13, lean=True)
    assert np.array_equal(a.row_ptr, b.row_ptr) and np.array_equal(a.col, b.col)


@pytest.mark.parametrize("omp", [False, True])
def test_levelsync_equals_queue_bfs(omp):
    """The level-synchronous BFS (plain and OpenMP builds) returns the FIFO-queue
    BFS levels: the level sets of a BFS are unique (Alg 1 P:330-334 drives the
    GPU level by level)."""
    cases = [inputs.rmat(16), inputs.random_graph(20000, 60000, 3), inputs.path(5000), inputs.in_star(1000),
             inputs.out_star(1000), inputs.twitter_like(n=1 << 16, m=1 << 20)]
    for g in cases:
        deg = np.diff(g.row_ptr)
        for src in {0, int(np.argmax(deg)), g.n - 1}:
            assert np.array_equal(oracle.bfs_levelsync(g.row_ptr, g.col, src, omp=omp),
                                  oracle.bfs(g.row_ptr, g.col, src))
    with pytest.raises(ValueError):
        oracle.bfs_levelsync(cases[0].row_ptr, cases[0].col, cases[0].n, omp=omp)
