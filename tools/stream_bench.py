"""Streamed-topology measurement (SURVEY 8(d) C4 at N = 1): RMAT-S pages live in
pinned host memory and every sweep streams them through the device ring.

Reports PageRank s/iter, BFS GTEPS and WCC time, each with the achieved
host->device GB/s against the pinned H2D bandwidth measured here (256 MiB
cudaMemcpyAsync, best of 10), as one JSON line.

    python tools/stream_bench.py --scale 30 [--iters 3]
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


def h2d_peak():
    src = torch.empty(256 << 20, dtype=torch.uint8, pin_memory=True)
    dst = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    best = 0.0
    for _ in range(10):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        dst.copy_(src, non_blocking=True)
        b.record()
        b.synchronize()
        best = max(best, (256 << 20) / (a.elapsed_time(b) * 1e-3) / 1e9)
    return best


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--scale", type=int, default=30)
    ap.add_argument("--iters", type=int, default=3)
    ap.add_argument("--ring", type=int, default=4)
    ap.add_argument("--batch", type=int, default=0)
    a = ap.parse_args()
    t0 = time.time()
    g = inputs.rmat(a.scale, lean=True)
    n, m = g.n, g.m
    deg = np.diff(g.row_ptr)
    t_gen = time.time() - t0
    t0 = time.time()
    gr = G.gts_build_pages(g.row_ptr, g.col)
    t_build = time.time() - t0
    del g
    st = gr.stats()
    peak = h2d_peak()
    ctx = G.gts_context_create(0)
    kw = dict(residency=G.GTS_STREAMED, ring_slots=a.ring, batch_pages=a.batch, timing=True)
    out = {}
    t0 = time.time()
    pr, s = G.gts_pagerank(ctx, gr, 1, out=torch.empty(n, dtype=torch.float32, device="cuda"), **kw)   # pins pages
    out["pin_and_first_iter_s"] = time.time() - t0
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
    ev[0].record()
    _, s = G.gts_pagerank(ctx, gr, a.iters, out=torch.empty(n, dtype=torch.float32, device="cuda"), **kw)
    ev[1].record()
    ev[1].synchronize()
    t = ev[0].elapsed_time(ev[1]) * 1e-3
    out["pagerank"] = {"s_per_iter": t / a.iters, "h2d_bytes": s["h2d_bytes"], "link_gbs": s["h2d_bytes"] / t / 1e9,
                       "link_frac": s["h2d_bytes"] / t / 1e9 / peak, "kernel_s": s["main_kernel_s"],
                       "copy_s": s["h2d_s"]}
    lv = torch.empty(n, dtype=torch.int32, device="cuda")
    ev[0].record()
    _, s = G.gts_bfs(ctx, gr, 0, out=lv, **kw)
    ev[1].record()
    ev[1].synchronize()
    t = ev[0].elapsed_time(ev[1]) * 1e-3
    out["bfs"] = {"s": t, "gteps": s["edges_traversed"] / t / 1e9, "nominal_gteps": m / t / 1e9,
                  "levels": s["levels_or_iters"], "h2d_bytes": s["h2d_bytes"],
                  "link_gbs": s["h2d_bytes"] / t / 1e9, "link_frac": s["h2d_bytes"] / t / 1e9 / peak,
                  "pages_processed": s["pages_processed"]}
    lab = torch.empty(n, dtype=torch.int32, device="cuda")
    ev[0].record()
    _, s = G.gts_wcc(ctx, gr, out=lab, **kw)
    ev[1].record()
    ev[1].synchronize()
    t = ev[0].elapsed_time(ev[1]) * 1e-3
    out["wcc"] = {"s": t, "sweeps": s["levels_or_iters"], "h2d_bytes": s["h2d_bytes"],
                  "link_gbs": s["h2d_bytes"] / t / 1e9, "link_frac": s["h2d_bytes"] / t / 1e9 / peak}
    line = {"workload": f"rmat{a.scale}_streamed", "n": n, "m": m, "topo_bytes": st["topo_bytes"],
            "num_pages": st["num_pages"], "h2d_peak_gbs": peak, "gen_s": t_gen, "build_s": t_build,
            "ring": a.ring, "batch_pages": a.batch or "default", **out}
    print(json.dumps(line), flush=True)
    ctx.free()


if __name__ == "__main__":
    main()
