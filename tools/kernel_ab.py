"""Kernel timing of the hot path on one graph (a development tool, not a bench line).

Builds degree-ordered RMAT-S pages once and runs each algorithm `--reps` times
through the C ABI with GTS_RUN_TIMING, printing the median main-kernel time
(CUDA events inside libgts) and call time per algorithm as one JSON line each.

    python tools/kernel_ab.py --scale 27 --algos pr,bfs,sssp,wcc --reps 3
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
ap.add_argument("--algos", default="pr,bfs,sssp,wcc")
ap.add_argument("--tag", default="")
ap.add_argument("--tunes", default="",
                help='gts_run_config tuning variants (gts.TUNABLE fields): "name:field=v,field2=w;name2:..."')
ap.add_argument("--variants", default="",
                help='A/B of development switches read by libgts at call time: "name:ENV=V,ENV2=W;name2:..."')
a = ap.parse_args()

g = inputs.rmat(a.scale)
algos = a.algos.split(",")
gr = G.gts_build_pages(g.row_ptr, g.col, order=True)
grw = G.gts_build_pages(g.row_ptr, g.col, inputs.edge_weights(g), order=True) if "sssp" in algos else None
ctx = G.gts_context_create(0)
import torch  # noqa: E402
try:   # the persisting-L2 limits the access-policy windows are clipped to
    from cuda.bindings import runtime as rt
    _, pmax = rt.cudaDeviceGetAttribute(rt.cudaDeviceAttr.cudaDevAttrMaxPersistingL2CacheSize, 0)
    _, wmax = rt.cudaDeviceGetAttribute(rt.cudaDeviceAttr.cudaDevAttrMaxAccessPolicyWindowSize, 0)
    print(json.dumps({"l2_bytes": torch.cuda.get_device_properties(0).L2_cache_size,
                      "persisting_l2_max_bytes": pmax, "access_policy_window_max_bytes": wmax}), flush=True)
except Exception as e:  # pragma: no cover
    print(json.dumps({"l2_probe_error": repr(e)}), flush=True)
n = g.n
dev_u = torch.empty(n, dtype=torch.int32, device="cuda")
dev_f = torch.empty(n, dtype=torch.float32, device="cuda")
variants = [v.partition(":") for v in a.variants.split(";")] if a.variants else [(a.tag, "", "")]
tunes = [t.partition(":") for t in a.tunes.split(";")] if a.tunes else []
# every tuning variant runs with the build as is (no environment switches)
variants = [(tag, "", "", {}) for tag, _, envs in variants if not envs] + \
           [(tag, "", envs, {}) for tag, _, envs in variants if envs] + \
           [(tag, "", "", dict(kv.split("=") for kv in filter(None, tv.split(",")))) for tag, _, tv in tunes]
for tag, _, envs, tune in variants:
    keys = []
    for kv in filter(None, envs.split(",")):
        k, v = kv.split("=")
        os.environ[k] = v
        keys.append(k)
    for al in algos:
        ks, cs, st = [], [], None
        for _ in range(a.reps + 1):
            if al == "pr":
                _, st = G.gts_pagerank(ctx, gr, 10, 0.85, out=dev_f, timing=True, tune=tune)
            elif al == "bfs":
                _, st = G.gts_bfs(ctx, gr, 0, out=dev_u, timing=True, tune=tune)
            elif al == "sssp":
                _, st = G.gts_sssp(ctx, grw, 0, out=dev_u, timing=True, tune=tune)
            else:
                _, st = G.gts_wcc(ctx, gr, out=dev_u, timing=True, tune=tune)
            ks.append(st["main_kernel_s"])
            cs.append(st["wall_s"])
        ks, cs = sorted(ks[1:]), sorted(cs[1:])
        per = 10 if al == "pr" else 1
        print(json.dumps({"tag": tag, "algo": al, "scale": a.scale, "main_kernel_ms": 1e3 * ks[len(ks) // 2] / per,
                          "per": "iteration" if per == 10 else "call", "call_ms": 1e3 * cs[len(cs) // 2],
                          "all_kernel_ms": [round(1e3 * k / per, 3) for k in ks], "edges": st["edges_traversed"],
                          "levels": st["levels_or_iters"], "finish_ms": 1e3 * st["finish_s"] / per}), flush=True)
    for k in keys:
        del os.environ[k]
