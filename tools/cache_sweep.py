"""Topology-cache size sweep for streamed BFS (the paper's Fig 11, P:1282;
cachedPIDMap, P:312 and Alg 1 lines 8/16/29).

Pages are streamed from pinned host memory; pages touched at an earlier level
stay in a device LRU cache of `cache_mib` MiB.  For each size: BFS time, H2D
bytes, and the hit rate next to the paper's naive estimate B / (S + L)
(B = cached pages).  One JSON line.

    python tools/cache_sweep.py --scales 27,28
"""
import argparse
import json
import os
import statistics
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import inputs  # noqa: E402
import paper_conf_sigmod_0002apsk16_b200 as G  # noqa: E402
from tools.stream_bench import h2d_peak  # noqa: E402

SIZES_MIB = [0, 32, 128, 512, 1024, 2048, 5120, 10240, 20480]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--scales", default="27")
    ap.add_argument("--reps", type=int, default=2)
    a = ap.parse_args()
    peak = h2d_peak()
    ctx = G.gts_context_create(0)
    rows = []
    for scale in [int(s) for s in a.scales.split(",")]:
        t0 = time.time()
        g = inputs.rmat(scale)
        n = g.n
        gr = G.gts_build_pages(g.row_ptr, g.col)
        del g
        st = gr.stats()
        topo_mib = st["topo_bytes"] / 2**20
        print(f"[cache_sweep] rmat{scale}: {st['num_pages']} pages ({topo_mib:.0f} MiB), built in "
              f"{time.time() - t0:.0f} s", file=sys.stderr, flush=True)
        lv = torch.empty(n, dtype=torch.int32, device="cuda")
        G.gts_bfs(ctx, gr, 0, out=lv, residency=G.GTS_STREAMED)         # registers the pinned pages
        for mib in SIZES_MIB:
            if mib > 2 * topo_mib:
                continue
            ws, last = [], None
            for _ in range(a.reps):
                ctx.evict(gr)                                           # drops the cache: every run starts cold
                _, s = G.gts_bfs(ctx, gr, 0, out=lv, residency=G.GTS_STREAMED, cache_mib=mib)
                ws.append(s["wall_s"])
                last = s
            w = statistics.median(ws)
            looks = last["cache_hits"] + last["cache_misses"]
            cached_pages = min(mib * 2**20 // st["page_bytes"], st["num_pages"])
            rows.append({"scale": scale, "cache_mib": mib, "s": w, "gteps": last["edges_traversed"] / w / 1e9,
                         "h2d_bytes": last["h2d_bytes"], "link_gbs": last["h2d_bytes"] / w / 1e9,
                         "page_visits": last["pages_processed"], "hits": last["cache_hits"],
                         "hit_rate": (last["cache_hits"] / looks) if looks else 0.0,
                         "naive_hit_rate": cached_pages / st["num_pages"]})
            print(f"[cache_sweep]   cache {mib:6d} MiB: {w:.3f} s, h2d {last['h2d_bytes'] / 1e9:.1f} GB, "
                  f"hit rate {rows[-1]['hit_rate']:.3f} (naive {rows[-1]['naive_hit_rate']:.3f})",
                  file=sys.stderr, flush=True)
        ctx.evict(gr)
        gr.free()
        del lv
        torch.cuda.empty_cache()
    print(json.dumps({"workload": "streamed_bfs_cache_sweep", "h2d_peak_gbs": peak, "rows": rows}))
    ctx.free()


if __name__ == "__main__":
    main()
