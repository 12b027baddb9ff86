"""Wall vs kernel time of gts_pagerank calls (1 and 10 iterations) on RMAT-27, device outputs."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import inputs  # noqa: E402
import paper_conf_sigmod_0002apsk16_b200 as G  # noqa: E402

g = inputs.rmat(int(sys.argv[1]) if len(sys.argv) > 1 else 27)
gr = G.gts_build_pages(g.row_ptr, g.col, order=True)
ctx = G.gts_context_create(0)
x = torch.empty(g.n, dtype=torch.float32, device="cuda")
G.gts_pagerank(ctx, gr, 1, out=x)
for env in ({}, {"GTS_L2_RESET": "0"}, {"GTS_L2_PERSIST": "0"}, {"GTS_PR_BIG": "1"}, {"GTS_PR_BIG": "1", "GTS_L2_RESET": "0"}):
    for k, v in env.items():
        os.environ[k] = v
    for it in (1, 10):
        torch.cuda.synchronize()
        t = time.perf_counter()
        _, st = G.gts_pagerank(ctx, gr, it, out=x, timing=True)
        w = time.perf_counter() - t
        print(env, it, f"wall {w*1e3:.2f} ms  scatter {st['main_kernel_s']*1e3:.2f} ms  finish {st['finish_s']*1e3:.2f} ms", flush=True)
    for k in env:
        del os.environ[k]
