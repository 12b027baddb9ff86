"""Ring-depth / batch sweep of the page streamer (the paper's Fig 10 axis, P:1206:
"#streams 1..32").  For each (ring_slots, batch_pages)
streamed PageRank iterations are timed and the achieved host->device rate is
reported against the pinned H2D peak measured here.  One JSON line.

    python tools/stream_sweep.py --scale 27
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import inputs  # noqa: E402
import paper_conf_sigmod_0002apsk16_b200 as G  # noqa: E402
from tools.stream_bench import h2d_peak  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--scale", type=int, default=27)
    ap.add_argument("--iters", type=int, default=2)
    a = ap.parse_args()
    g = inputs.rmat(a.scale)
    gr = G.gts_build_pages(g.row_ptr, g.col, order=True)
    n = g.n
    del g
    peak = h2d_peak()
    ctx = G.gts_context_create(0)
    x = torch.empty(n, dtype=torch.float32, device="cuda")
    G.gts_pagerank(ctx, gr, 1, out=x, residency=G.GTS_STREAMED)       # pin pages once
    res = []
    for ring in (1, 2, 4, 8, 16, 32):
        for batch in (1, 8, 32, 64, 128):
            if ring * batch > 2048:
                continue
            ev = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
            ev[0].record()
            _, st = G.gts_pagerank(ctx, gr, a.iters, out=x, residency=G.GTS_STREAMED, ring_slots=ring,
                                   batch_pages=batch)
            ev[1].record()
            ev[1].synchronize()
            t = ev[0].elapsed_time(ev[1]) * 1e-3
            res.append({"ring": ring, "batch_pages": batch, "s_per_iter": t / a.iters,
                        "link_gbs": st["h2d_bytes"] / t / 1e9, "link_frac": st["h2d_bytes"] / t / 1e9 / peak})
    print(json.dumps({"workload": f"rmat{a.scale}_streamed_pagerank", "h2d_peak_gbs": peak, "sweep": res}))
    ctx.free()


if __name__ == "__main__":
    main()
