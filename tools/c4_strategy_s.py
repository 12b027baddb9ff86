"""BASELINE configs[3] (C4) on one B200: RMAT-30 (n = 2^30, m = 2^34, 83 GB of pages),
topology streamed from pinned host memory, Strategy-S.

One GPU runs the N-rank job through virtual ranks: each rank streams only its own
pages (its contiguous range, ~T_topo / N) and keeps only its WA range, and remote
updates go straight into the owner's WA (GTS_ROUTE_PEER; message routing would need
8 B per remote edge of buffers).  The ranks run one after another, so the time is
the N-GPU job's work done on one GPU, not an N-GPU time; what it shows is the
C4 path at full size: results equal to the single-rank run (BFS bit-exact,
PageRank within the 1e-4 gate of it), host-link rate, per-rank WA bytes.

    python tools/c4_strategy_s.py --scale 30 --ranks 1,2,4
"""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import inputs  # noqa: E402
import paper_conf_sigmod_0002apsk16_b200 as G  # noqa: E402
from tools.stream_bench import h2d_peak  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--scale", type=int, default=30)
    ap.add_argument("--ranks", default="1,2,4")
    ap.add_argument("--iters", type=int, default=2)
    a = ap.parse_args()
    t0 = time.time()
    g = inputs.rmat(a.scale, lean=True)
    n, m = g.n, g.m
    t_gen = time.time() - t0
    t0 = time.time()
    gr = G.gts_build_pages(g.row_ptr, g.col)
    t_build = time.time() - t0
    del g
    st = gr.stats()
    peak = h2d_peak()
    ctx = G.gts_context_create(0)
    base = dict(residency=G.GTS_STREAMED, timing=True)
    G.gts_pagerank(ctx, gr, 1, 0.85, **base)     # warm-up: pins the 83 GB of host pages once
    ref_lv = ref_pr = None
    rows = []
    lv = torch.empty(n, dtype=torch.int32, device="cuda")
    pr = torch.empty(n, dtype=torch.float32, device="cuda")
    for N in [int(x) for x in a.ranks.split(",")]:
        kw = dict(base)
        if N > 1:
            kw.update(strategy=G.GTS_STRATEGY_S, virtual_ranks=N, route_peer=True)
        t0 = time.perf_counter()
        _, sb = G.gts_bfs(ctx, gr, 0, out=lv, **kw)
        t_bfs = time.perf_counter() - t0
        t0 = time.perf_counter()
        _, sp = G.gts_pagerank(ctx, gr, a.iters, 0.85, out=pr, **kw)
        t_pr = (time.perf_counter() - t0) / a.iters
        lv_h = lv.cpu().numpy().view(np.uint32)
        pr_h = pr.cpu().numpy().astype(np.float64)
        if ref_lv is None:
            ref_lv, ref_pr = lv_h.copy(), pr_h.copy()
            same_bfs, pr_rel = True, 0.0
        else:
            same_bfs = bool(np.array_equal(lv_h, ref_lv))
            pr_rel = float(np.max(np.abs(pr_h - ref_pr) / ref_pr))
        row = {"ranks": N, "strategy": "S (peer)" if N > 1 else "single", "bfs_s": t_bfs,
               "bfs_gteps": sb["edges_traversed"] / t_bfs / 1e9, "bfs_h2d_gbs": sb["h2d_bytes"] / t_bfs / 1e9,
               "pr_s_per_iter": t_pr, "pr_h2d_gbs": sp["h2d_bytes"] / a.iters / t_pr / 1e9,
               "h2d_peak_gbs": peak, "pr_link_frac": sp["h2d_bytes"] / a.iters / t_pr / 1e9 / peak,
               "wa_bytes_per_rank_pr": sp["wa_bytes"], "wa_bytes_per_rank_bfs": sb["wa_bytes"],
               "bfs_equal_to_single": same_bfs, "pr_max_rel_vs_single": pr_rel}
        rows.append(row)
        print(json.dumps(row), flush=True)
    print(json.dumps({"workload": f"rmat{a.scale}_streamed_strategy_s", "n": n, "m": m, "topo_bytes": st["topo_bytes"],
                      "gen_s": t_gen, "build_s": t_build, "rows": rows}))


if __name__ == "__main__":
    main()
