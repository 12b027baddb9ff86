"""Run selected GTS algorithms once on RMAT-S (for ncu captures; not a benchmark)."""
import argparse
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import inputs  # noqa: E402
import paper_conf_sigmod_0002apsk16_b200 as G  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--scale", type=int, default=27)
ap.add_argument("--algos", default="bfs,pr")
ap.add_argument("--pr-iters", type=int, default=2)
ap.add_argument("--page-bytes", type=int, default=1 << 20)
ap.add_argument("--reps", type=int, default=1)
ap.add_argument("--relabel", action="store_true")
ap.add_argument("--order", action="store_true")
ap.add_argument("--streamed", action="store_true")
a = ap.parse_args()
t = time.time()
g = inputs.rmat(a.scale)
src = 0
if a.relabel:
    p = inputs.indegree_order(g)
    src = int(p[0])
    g = inputs.permute(g, p)
    print("relabelled", time.time() - t, flush=True)
w = inputs.edge_weights(g) if "sssp" in a.algos else None
gr = G.gts_build_pages(g.row_ptr, g.col, page_bytes=a.page_bytes, order=a.order)
grw = G.gts_build_pages(g.row_ptr, g.col, w, page_bytes=a.page_bytes, order=a.order) if w is not None else None
print("built", time.time() - t, flush=True)
ctx = G.gts_context_create(0)
kw = dict(residency=G.GTS_STREAMED) if a.streamed else {}
for _ in range(a.reps):
    for algo in a.algos.split(","):
        if algo == "bfs":
            _, st = G.gts_bfs(ctx, gr, src, timing=True, **kw)
        elif algo == "pr":
            _, st = G.gts_pagerank(ctx, gr, a.pr_iters, timing=True, **kw)
        elif algo == "sssp":
            _, st = G.gts_sssp(ctx, grw, src, timing=True, **kw)
        elif algo == "wcc":
            _, st = G.gts_wcc(ctx, gr, timing=True, **kw)
        print(algo, st, flush=True)
