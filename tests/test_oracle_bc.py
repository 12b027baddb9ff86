"""Pins for oracle.bc (Brandes betweenness from a set of sources; BC is run on
GTS in the paper, Fig 13c).  Checked against networkx
betweenness_centrality_subset (a different implementation of the same sum over
source/target pairs of sigma_st(v)/sigma_st), brute-force enumeration of all
shortest paths on tiny graphs (multi-edges included), and closed forms."""
import itertools

import networkx as nx
import numpy as np
import pytest

import inputs
import oracle


def brute_bc(n, edges, sources):
    """sum over s in sources, t != s reachable, of (#shortest s-t paths through v) / (#shortest s-t paths),
    by explicit enumeration of edge sequences (parallel edges are distinct paths)."""
    adj = [[] for _ in range(n)]
    for u, v in edges:
        adj[u].append(v)
    bc = np.zeros(n)
    for s in sources:
        lv = oracle.bfs(*_csr(n, edges), s)
        paths = {s: [[s]]}
        for L in range(1, n):
            for w in range(n):
                if lv[w] != L:
                    continue
                paths[w] = [p + [w] for u in range(n) if lv[u] == L - 1 for p in paths[u] for x in adj[u] if x == w]
        for t, ps in paths.items():
            if t == s:
                continue
            for v in range(n):
                if v in (s, t):
                    continue
                bc[v] += sum(1 for p in ps if v in p) / len(ps)
    return bc


def _csr(n, edges):
    g = inputs.from_edges(n, edges)
    return g.row_ptr, g.col


def test_bc_brute_force_tiny():
    rng = np.random.default_rng(5)
    for _ in range(60):
        n = int(rng.integers(2, 7))
        m = int(rng.integers(0, 3 * n))
        edges = [tuple(e) for e in rng.integers(0, n, size=(m, 2)).tolist()]
        g = inputs.from_edges(n, edges)
        srcs = sorted(set(rng.integers(0, n, size=2).tolist()))
        assert np.allclose(oracle.bc(g.row_ptr, g.col, srcs), brute_bc(n, edges, srcs), atol=1e-12)


def test_bc_vs_networkx():
    g = inputs.random_graph(300, 1500, 3, self_loops=False)
    src_of = np.repeat(np.arange(g.n), np.diff(g.row_ptr).astype(np.int64))
    pairs = sorted(set(zip(src_of.tolist(), g.col.tolist())))
    g = inputs.from_edges(g.n, pairs)
    G = nx.DiGraph()
    G.add_nodes_from(range(g.n))
    G.add_edges_from(pairs)
    srcs = [0, 5, 17, 100]
    ref = nx.betweenness_centrality_subset(G, sources=srcs, targets=list(range(g.n)), normalized=False)
    got = oracle.bc(g.row_ptr, g.col, srcs)
    assert max(abs(got[v] - ref[v]) for v in range(g.n)) < 1e-9


def test_bc_closed_forms():
    n = 50
    g = inputs.path(n)              # source 0: every v in 1..n-2 lies on the paths to the n-1-v later vertices
    assert np.allclose(oracle.bc(g.row_ptr, g.col, [0]), [0] + [n - 1 - v for v in range(1, n)])
    g = inputs.out_star(20)          # leaves are endpoints only
    assert np.allclose(oracle.bc(g.row_ptr, g.col, [0]), 0)
    # diamond 0->{1,2}->3: two shortest paths to 3, each middle vertex carries half
    g = inputs.from_edges(4, [(0, 1), (0, 2), (1, 3), (2, 3)])
    assert np.allclose(oracle.bc(g.row_ptr, g.col, [0]), [0, 0.5, 0.5, 0])
    # a doubled edge 0->1 doubles sigma(1) but leaves the dependency ratio unchanged
    g = inputs.from_edges(4, [(0, 1), (0, 1), (0, 2), (1, 3), (2, 3)])
    assert np.allclose(oracle.bc(g.row_ptr, g.col, [0]), [0, 2 / 3, 1 / 3, 0])
