"""Where do slow calls lose their time?  Runs the bench step (BFS, PageRank, SSSP,
WCC on degree-ordered RMAT-S) repeatedly under torch.profiler and, per call,
compares the device busy time (sum of the call's kernels / memsets / copies,
CUPTI records) with its span; for the slowest calls it prints the largest idle
gaps on the device and the longest CUDA runtime API calls on the host.

    python tools/call_jitter.py --scale 27 --steps 20
"""
import argparse
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402
from torch.profiler import ProfilerActivity, profile, record_function  # noqa: E402

import inputs  # noqa: E402
import paper_conf_sigmod_0002apsk16_b200 as G  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--scale", type=int, default=27)
ap.add_argument("--steps", type=int, default=20)
a = ap.parse_args()
g = inputs.rmat(a.scale)
gr = G.gts_build_pages(g.row_ptr, g.col, order=True)
w = inputs.edge_weights(g)
grw = G.gts_build_pages(g.row_ptr, g.col, w, order=True)
n = g.n
del g, w
ctx = G.gts_context_create(0)
s = torch.cuda.current_stream()
ctx.set_stream(s.cuda_stream)
u = torch.empty(n, dtype=torch.int32, device="cuda")
f = torch.empty(n, dtype=torch.float32, device="cuda")
calls = {"bfs": lambda: G.gts_bfs(ctx, gr, 0, out=u, timing=True),
         "pr": lambda: G.gts_pagerank(ctx, gr, 10, 0.85, out=f, timing=True),
         "sssp": lambda: G.gts_sssp(ctx, grw, 0, out=u, timing=True),
         "wcc": lambda: G.gts_wcc(ctx, gr, out=u, timing=True)}
for _ in range(2):
    for c in calls.values():
        c()
torch.cuda.synchronize()
marks = []
with profile(activities=[ProfilerActivity.CPU, ProfilerActivity.CUDA]) as prof:
    for i in range(a.steps):
        for name, c in calls.items():
            t0 = time.perf_counter_ns()
            with record_function(f"call:{name}:{i}"):
                c()
            t1 = time.perf_counter_ns()
            marks.append((name, i, t0, t1))
    torch.cuda.synchronize()
evs = list(prof.events())
dev = sorted([e for e in evs if e.device_type == torch.autograd.DeviceType.CUDA], key=lambda e: e.time_range.start)
cpu = [e for e in evs if e.device_type == torch.autograd.DeviceType.CPU]
rng = {e.name: e for e in cpu if e.name.startswith("call:")}
api = [e for e in cpu if e.name.startswith("cuda") or e.name.startswith("cu")]
rows = []
for name, i, t0, t1 in marks:
    r = rng[f"call:{name}:{i}"]
    a0, a1 = r.time_range.start, r.time_range.end
    d = [e for e in dev if a0 <= e.time_range.start <= a1 + 2000]
    busy = sum(e.time_range.end - e.time_range.start for e in d)
    span = (d[-1].time_range.end - d[0].time_range.start) if d else 0
    gaps = []
    for x, y in zip(d, d[1:]):
        gaps.append((y.time_range.start - x.time_range.end, x.name[:40], y.name[:40]))
    gaps.sort(reverse=True)
    slow_api = sorted([(e.time_range.end - e.time_range.start, e.name) for e in api
                       if a0 <= e.time_range.start <= a1], reverse=True)[:4]
    rows.append((name, i, (t1 - t0) / 1e6, (a1 - a0) / 1e3, busy / 1e3, span / 1e3, gaps[:3], slow_api))
for name in calls:
    rr = [r for r in rows if r[0] == name]
    wall = np.array([r[2] for r in rr])
    print(f"{name}: host wall ms median {np.median(wall):.2f} max {wall.max():.2f}; device busy ms median "
          f"{np.median([r[4] for r in rr]):.2f} max {max(r[4] for r in rr):.2f}; span median "
          f"{np.median([r[5] for r in rr]):.2f} max {max(r[5] for r in rr):.2f}")
    for r in sorted(rr, key=lambda r: -r[2])[:3]:
        print(f"   step {r[1]:2d}: wall {r[2]:.2f} ms busy {r[4]:.2f} span {r[5]:.2f}")
        for gp in r[6]:
            print(f"      gap {gp[0] / 1e3:8.3f} ms  {gp[1]} -> {gp[2]}")
        for ap_ in r[7]:
            print(f"      api {ap_[0] / 1e3:8.3f} ms  {ap_[1]}")
