"""A/B timing of PageRank scatter variants on one graph (not a benchmark line).

Builds degree-ordered RMAT-S pages once, then for each variant (a set of GTS_*
environment switches read by libgts at call time) runs 10-iteration PageRank
`--reps` times and prints the median scatter-kernel time per iteration and the
max relative difference to the first variant's ranks.

    python tools/pr_variants.py --scale 27 --variants "base:;fixall:GTS_PR_FIX=1;fixmix:GTS_PR_FIX=2"
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

import inputs  # noqa: E402
import paper_conf_sigmod_0002apsk16_b200 as G  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--scale", type=int, default=27)
ap.add_argument("--reps", type=int, default=3)
ap.add_argument("--iters", type=int, default=10)
ap.add_argument("--variants", default="base:;fixall:GTS_PR_FIX=1;fixmix:GTS_PR_FIX=2")
ap.add_argument("--out", default=None)
a = ap.parse_args()

g = inputs.rmat(a.scale)
gr = G.gts_build_pages(g.row_ptr, g.col, order=True)
ctx = G.gts_context_create(0)
res, first = {}, None
for spec in a.variants.split(";"):
    name, _, envs = spec.partition(":")
    keys = []
    for kv in filter(None, envs.split(",")):
        k, v = kv.split("=")
        os.environ[k] = v
        keys.append(k)
    t = []
    for _ in range(a.reps + 1):
        x, st = G.gts_pagerank(ctx, gr, a.iters, timing=True)
        t.append(st["main_kernel_s"] / a.iters)
    t = sorted(t[1:])
    if first is None:
        first = x.astype(np.float64)
    rel = float(np.max(np.abs(x - first) / first))
    res[name] = dict(env=envs, scatter_ms=1e3 * t[len(t) // 2], all_ms=[1e3 * v for v in t], max_rel_vs_first=rel,
                     sum=float(np.sum(x, dtype=np.float64)))
    print(name, json.dumps(res[name]), flush=True)
    for k in keys:
        del os.environ[k]
if a.out:
    with open(a.out, "w") as f:
        json.dump(dict(scale=a.scale, iters=a.iters, variants=res), f, indent=1)
