"""Per-call breakdown of the bench step (BFS, PR, SSSP, WCC on degree-ordered
RMAT-S, device outputs): host wall, kernel, finish, merge, upload per call."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import inputs  # noqa: E402
import paper_conf_sigmod_0002apsk16_b200 as G  # noqa: E402

scale = int(sys.argv[1]) if len(sys.argv) > 1 else 27
g = inputs.rmat(scale)
gr = G.gts_build_pages(g.row_ptr, g.col, order=True)
grw = G.gts_build_pages(g.row_ptr, g.col, inputs.edge_weights(g), order=True)
n = g.n
del g
ctx = G.gts_context_create(0)
ctx.set_stream(torch.cuda.current_stream().cuda_stream)
o32 = torch.empty(n, dtype=torch.int32, device="cuda")
of = torch.empty(n, dtype=torch.float32, device="cuda")
for step in range(4):
    for name, fn in (("bfs", lambda: G.gts_bfs(ctx, gr, 0, out=o32, timing=True)),
                     ("pr", lambda: G.gts_pagerank(ctx, gr, 10, out=of, timing=True)),
                     ("sssp", lambda: G.gts_sssp(ctx, grw, 0, out=o32, timing=True)),
                     ("wcc", lambda: G.gts_wcc(ctx, gr, out=o32, timing=True))):
        torch.cuda.synchronize()
        t = time.perf_counter()
        _, st = fn()
        torch.cuda.synchronize()
        w = time.perf_counter() - t
        print(f"step {step} {name:5s} wall {w*1e3:8.2f} ms  lib_wall {st['wall_s']*1e3:8.2f}  kern {st['main_kernel_s']*1e3:7.2f}"
              f"  fin {st['finish_s']*1e3:6.2f}  upload {st['upload_s']*1e3:7.2f}  iters {st['levels_or_iters']}", flush=True)
