"""Small end-to-end run of every kernel of libgts, for compute-sanitizer.

    compute-sanitizer --tool memcheck|racecheck|synccheck python tools/sanitize_run.py

RMAT-14 (1 MiB, 4 KiB and 256 B pages: SP, LP and LP-slicing paths), every
algorithm, natural and degree order, resident and streamed, one rank and 3
virtual ranks under P / S / S_BCAST; results checked against the oracle so a
run that "passes" the sanitizer also computed the right thing.
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

import inputs  # noqa: E402
import oracle  # noqa: E402
import paper_conf_sigmod_0002apsk16_b200 as G  # noqa: E402

scale = int(os.environ.get("GTS_SAN_SCALE", "14"))
quick = os.environ.get("GTS_SAN_QUICK", "0") == "1"     # racecheck: one call per kernel family
g = inputs.rmat(scale)
w = inputs.edge_weights(g)
want_bfs = oracle.bfs(g.row_ptr, g.col, 0)
want_sssp = oracle.sssp(g.row_ptr, g.col, w, 0)
want_wcc = oracle.wcc(g.row_ptr, g.col)
want_pr = oracle.pagerank(g.row_ptr, g.col, 10, 0.85)
ctx = G.gts_context_create(0)
runs = 0
for pb in ((4096,) if quick else (1 << 20, 4096, 256)):
    for order in ((True,) if quick else (False, True)):
        gr = G.gts_build_pages(g.row_ptr, g.col, page_bytes=pb, order=order)
        grw = G.gts_build_pages(g.row_ptr, g.col, w, page_bytes=max(pb, 512), order=order)
        grs = G.gts_build_pages(g.row_ptr, g.col, page_bytes=pb, order=order, symmetric=True)
        for res in ((G.GTS_RESIDENT,) if quick else (G.GTS_RESIDENT, G.GTS_STREAMED)):
            for strat, V in (((0, 0), (1, 2)) if quick else ((0, 0), (0, 3), (1, 3), (2, 3))):
                kw = dict(residency=res, strategy=strat, virtual_ranks=V, batch_pages=4, ring_slots=2)
                lv, _ = G.gts_bfs(ctx, gr, 0, **kw)
                assert np.array_equal(lv, want_bfs), ("bfs", pb, order, res, strat, V)
                d, _ = G.gts_sssp(ctx, grw, 0, **kw)
                assert np.array_equal(d, want_sssp), ("sssp", pb, order, res, strat, V)
                lab, _ = G.gts_wcc(ctx, grs if strat == 1 else gr, **kw)
                assert np.array_equal(lab, want_wcc), ("wcc", pb, order, res, strat, V)
                x, _ = G.gts_pagerank(ctx, gr, 10, 0.85, **kw)
                assert np.max(np.abs(x - want_pr) / want_pr) <= 1e-4, ("pr", pb, order, res, strat, V)
                runs += 4
        if pb == 4096:
            for micro in ("edge", "vertex", "hybrid"):
                assert np.array_equal(G.gts_bfs(ctx, gr, 0, micro=micro)[0], want_bfs)
                G.gts_pagerank(ctx, gr, 10, 0.85, micro=micro)
                runs += 2
            bc, _ = G.gts_bc(ctx, gr, [0, 5])
            assert np.allclose(bc, oracle.bc(g.row_ptr, g.col, [0, 5]), rtol=1e-9, atol=1e-9)
            G.gts_bfs(ctx, gr, 0, residency=G.GTS_STREAMED, cache_mib=1)
            runs += 2
ctx.free()
print(f"sanitize_run: {runs} calls on RMAT-{scale}, all results equal to the oracle")
