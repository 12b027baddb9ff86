"""Device timeline of one gts_bfs call (degree-ordered RMAT-S, device output):
every kernel / memset / memcpy the call issues, with its start offset, duration
and the idle gap before it, from the CUPTI activity records torch.profiler
collects (they cover libgts's launches, not only torch's).

    python tools/bfs_timeline.py [scale] [algo: bfs|sssp|wcc|pr]
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
from torch.profiler import ProfilerActivity, profile  # noqa: E402

import inputs  # noqa: E402
import paper_conf_sigmod_0002apsk16_b200 as G  # noqa: E402

scale = int(sys.argv[1]) if len(sys.argv) > 1 else 27
algo = sys.argv[2] if len(sys.argv) > 2 else "bfs"
g = inputs.rmat(scale)
w = inputs.edge_weights(g) if algo == "sssp" else None
gr = G.gts_build_pages(g.row_ptr, g.col, w, order=True)
n = g.n
del g
ctx = G.gts_context_create(0)
ctx.set_stream(torch.cuda.current_stream().cuda_stream)
out = torch.empty(n, dtype=torch.float32 if algo == "pr" else torch.int32, device="cuda")
call = {"bfs": lambda: G.gts_bfs(ctx, gr, 0, out=out),
        "sssp": lambda: G.gts_sssp(ctx, gr, 0, out=out),
        "wcc": lambda: G.gts_wcc(ctx, gr, out=out),
        "pr": lambda: G.gts_pagerank(ctx, gr, 10, out=out)}[algo]
for _ in range(3):
    call()
torch.cuda.synchronize()
with profile(activities=[ProfilerActivity.CPU, ProfilerActivity.CUDA]) as prof:
    call()
    torch.cuda.synchronize()
ev = [e for e in prof.events() if e.device_type == torch.autograd.DeviceType.CUDA]
ev.sort(key=lambda e: e.time_range.start)
t0 = ev[0].time_range.start
prev_end = t0
busy = 0.0
print(f"{algo} RMAT-{scale}: {len(ev)} device activities")
print(f"{'start_us':>10} {'dur_us':>9} {'gap_us':>8}  name")
for e in ev:
    s, d = e.time_range.start, e.time_range.end - e.time_range.start
    print(f"{s - t0:10.1f} {d:9.1f} {s - prev_end:8.1f}  {e.name[:90]}")
    busy += d
    prev_end = max(prev_end, e.time_range.end)
print(f"span {prev_end - t0:.1f} us, busy {busy:.1f} us, idle {prev_end - t0 - busy:.1f} us")
