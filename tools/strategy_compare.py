"""Strategy-P vs Strategy-S vs S_BCAST per rank (the paper's Fig 9 comparison,
P:1120-1200), from virtual ranks on one GPU.

One GPU cannot time N GPUs, so this records what each strategy makes a rank do
and move, which the times on N GPUs follow: pages processed per rank, edges
traversed, merge bytes per rank (what crosses NVLink), routed messages, device
WA bytes per rank, and host page bytes per rank (owner-filtered builds).  The
cost model's t_sync(N) (Eq 1) is estimated from the merge bytes at
the NVLink 5 bandwidth (900 GB/s per direction) -- a model, labelled as such.

    python tools/strategy_compare.py --scale 22 --ranks 2,4,8
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

import inputs  # noqa: E402
import paper_conf_sigmod_0002apsk16_b200 as G  # noqa: E402

NVLINK_GBS = 900.0

ap = argparse.ArgumentParser()
ap.add_argument("--scale", type=int, default=22)
ap.add_argument("--ranks", default="2,4,8")
a = ap.parse_args()
g = inputs.rmat(a.scale)
gr = G.gts_build_pages(g.row_ptr, g.col, order=True)
grs = G.gts_build_pages(g.row_ptr, g.col, order=True, symmetric=True)
topo = gr.stats()["topo_bytes"]
ctx = G.gts_context_create(0)
rows = []
names = {0: "P", 1: "S", 2: "S_BCAST"}
_, s1 = G.gts_bfs(ctx, gr, 0, timing=True)
_, p1 = G.gts_pagerank(ctx, gr, 10, 0.85, timing=True)
rows.append({"N": 1, "strategy": "single", "bfs_kernel_s": s1["main_kernel_s"], "pr_kernel_s_per_iter": p1["main_kernel_s"] / 10,
             "bfs_pages": s1["pages_processed"], "pr_pages_per_iter": p1["pages_processed"] / 10})
for N in [int(x) for x in a.ranks.split(",")]:
    for strat in (0, 1, 2):
        hb = [G.gts_build_pages(g.row_ptr, g.col, order=True, owner=(r, N, strat)).stats()["host_page_bytes"]
              for r in range(N)]
        _, sb = G.gts_bfs(ctx, gr, 0, strategy=strat, virtual_ranks=N, timing=True)
        _, sp = G.gts_pagerank(ctx, gr, 10, 0.85, strategy=strat, virtual_ranks=N, timing=True)
        _, sw = G.gts_wcc(ctx, grs if strat == 1 else gr, strategy=strat, virtual_ranks=N, timing=True)
        row = {"N": N, "strategy": names[strat],
               "bfs_pages_per_rank": sb["pages_processed"] / N, "bfs_edges_per_rank": sb["edges_traversed"] / N,
               "bfs_merge_bytes_per_rank": sb["nccl_bytes"] / N, "bfs_routed_msgs": sb["routed_msgs"],
               "bfs_levels": sb["levels_or_iters"], "bfs_wa_bytes_per_rank": sb["wa_bytes"],
               "pr_pages_per_rank_per_iter": sp["pages_processed"] / N / 10,
               "pr_merge_bytes_per_rank_per_iter": sp["nccl_bytes"] / N / 10,
               "pr_routed_msgs_per_iter": sp["routed_msgs"] / 10, "pr_wa_bytes_per_rank": sp["wa_bytes"],
               "wcc_rounds": sw["levels_or_iters"], "wcc_merge_bytes_per_rank": sw["nccl_bytes"] / N,
               "host_page_bytes_per_rank_max": max(hb), "topo_bytes": topo,
               "model_t_sync_pr_per_iter_s": sp["nccl_bytes"] / N / 10 / (NVLINK_GBS * 1e9),
               "model_t_sync_bfs_s": sb["nccl_bytes"] / N / (NVLINK_GBS * 1e9)}
        rows.append(row)
        print(json.dumps(row), flush=True)
print(json.dumps({"scale": a.scale, "n": g.n, "m": g.m, "rows": rows}))
