"""Micro-level technique x graph density sweep (the paper's Fig 14, App E
P:1580-1582): RMAT-28 with #vertices:#edges from 1:4 to
1:32, BFS and PageRank, each slotted page processed edge-centric (VWC, a warp
per vertex), vertex-centric (a thread per vertex), hybrid (per page by
density), and with the B200 defaults (tile engine for BFS, hot-set scatter for
PageRank; "tile" = the tile engine with plain REDs for PageRank).  Pages are
resident, natural VID order (as in the paper).  One JSON line.

    python tools/micro_sweep.py --scale 28 --efs 4,8,16,32
"""
import argparse
import json
import os
import statistics
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import inputs  # noqa: E402
import paper_conf_sigmod_0002apsk16_b200 as G  # noqa: E402

BFS_MICRO = ["edge", "vertex", "hybrid", "default"]
PR_MICRO = ["edge", "vertex", "hybrid", "tile", "default"]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--scale", type=int, default=28)
    ap.add_argument("--efs", default="4,8,16,32")
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--pr-iters", type=int, default=3)
    a = ap.parse_args()
    ctx = G.gts_context_create(0)
    rows = []
    for ef in [int(x) for x in a.efs.split(",")]:
        t0 = time.time()
        g = inputs.rmat(a.scale, edge_factor=ef, lean=ef >= 32)
        n, m = g.n, g.m
        gr = G.gts_build_pages(g.row_ptr, g.col)
        deg = np.diff(g.row_ptr)
        del g
        st = gr.stats()
        print(f"[micro_sweep] scale {a.scale} ef {ef}: built in {time.time() - t0:.0f} s, "
              f"{st['num_pages']} pages", file=sys.stderr, flush=True)
        lv = torch.empty(n, dtype=torch.int32, device="cuda")
        x = torch.empty(n, dtype=torch.float32, device="cuda")
        G.gts_bfs(ctx, gr, 0, out=lv)                       # upload once (excluded)
        trav = None
        for micro in BFS_MICRO:
            ks, ws = [], []
            for _ in range(a.reps + 1):
                _, s = G.gts_bfs(ctx, gr, 0, out=lv, timing=True, micro=micro)
                ks.append(s["main_kernel_s"])
                ws.append(s["wall_s"])
                trav = s["edges_traversed"]
            k, w = statistics.median(ks[1:]), statistics.median(ws[1:])
            rows.append({"ef": ef, "algo": "bfs", "micro": micro, "kernel_s": k, "call_s": w,
                         "gteps_kernel": trav / k / 1e9, "gteps_call": trav / w / 1e9})
            print(f"[micro_sweep]   bfs {micro:8s} kernels {k * 1e3:8.2f} ms  call {w * 1e3:8.2f} ms",
                  file=sys.stderr, flush=True)
        for micro in PR_MICRO:
            ks, ws = [], []
            for _ in range(a.reps + 1):
                _, s = G.gts_pagerank(ctx, gr, a.pr_iters, out=x, timing=True, micro=micro)
                ks.append(s["main_kernel_s"] / a.pr_iters)
                ws.append(s["wall_s"] / a.pr_iters)
            k, w = statistics.median(ks[1:]), statistics.median(ws[1:])
            rows.append({"ef": ef, "algo": "pagerank", "micro": micro, "kernel_s_per_iter": k, "call_s_per_iter": w,
                         "gteps_kernel": m / k / 1e9})
            print(f"[micro_sweep]   pr  {micro:8s} scatter {k * 1e3:8.2f} ms/iter  call {w * 1e3:8.2f} ms/iter",
                  file=sys.stderr, flush=True)
        rows.append({"ef": ef, "n": n, "m": m, "num_pages": st["num_pages"], "n_lp": st["n_lp"],
                     "max_outdeg": int(deg.max()), "bfs_edges_traversed": trav})
        ctx.evict(gr)
        gr.free()
        del lv, x
        torch.cuda.empty_cache()
    print(json.dumps({"workload": f"rmat{a.scale}_density_sweep", "page_bytes": 1 << 20, "order": "natural",
                      "rows": rows}))
    ctx.free()


if __name__ == "__main__":
    main()
