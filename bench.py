#!/usr/bin/env python
"""Benchmark of the GTS hot path on B200 (driver contract).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl gts|reference] [--scale S]

One step = one pass of the whole hot path over the resident RMAT-S graph
(default S = 27, BASELINE.json configs[2]): BFS from vertex 0, 10 PageRank
iterations, SSSP from vertex 0 (hashed weights), WCC.  `value` is BFS GTEPS
(edges traversed / BFS device time, all ranks' work / max-over-ranks time);
PageRank s/iter, SSSP and WCC seconds are reported beside it.  Inputs (the
9.8 GB topology) are larger than L2, so no flush is needed between steps.

N > 1: launched by torchrun, one process per GPU, Strategy-P (pages
partitioned h(j) = j mod N, WA merged by NCCL inside libgts).

--impl reference runs the oracle (the paper-defined CPU program of oracle/) on
the host cores as the reference arm (rank 0 only).
"""
from __future__ import annotations

import argparse
import gc
import json
import os
import shutil
import subprocess
import sys
import tempfile
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

FALLBACK_HBM_GBS = 6650.0
METRIC = "BFS GTEPS and PageRank s/iter on RMAT-27..30 at 1/2/4/8 B200; % HBM/link BW"


def log(*a):
    print(*a, file=sys.stderr, flush=True)


def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return FALLBACK_HBM_GBS, "fallback (B200_PROFILING.md)"


class ClockSampler:
    """SM clocks + throttle reasons during the timed region.

    Default (GTS_BENCH_CLOCKS=kick): in-process NVML, one sample taken by a helper
    thread each time the step starts its PageRank call (kick()), i.e. while the
    GPU is loaded and the host is not on the critical path: a poller running
    concurrently (nvidia-smi -lms 200, the "smi" mode) stalls the per-level host
    synchronisations of SSSP/WCC through the driver lock and measured +0-40 ms
    per call.  "nvml" polls in-process every 200 ms, "off" disables sampling."""
    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, device):
        self.device = device
        self.lines = []
        self.proc = None

    def start(self):
        mode = os.environ.get("GTS_BENCH_CLOCKS", "kick")
        if mode in ("nvml", "kick"):
            return self._start_nvml(kicked=mode == "kick")
        if mode == "off":
            return
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--query-gpu={self.FIELDS}", "--format=csv,noheader,nounits",
                                          "-lms", "200", "-i", str(self.device)], stdout=subprocess.PIPE,
                                         stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception as e:  # pragma: no cover
            log("clock sampler unavailable:", e)

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    # in-process NVML sampling (GTS_BENCH_CLOCKS=nvml): the same fields as the
    # nvidia-smi line, without a second process polling the driver
    def kick(self):
        if getattr(self, "kick_ev", None) is not None:
            self.kick_ev.set()

    def _start_nvml(self, kicked=False):
        try:
            import pynvml
            pynvml.nvmlInit()
        except Exception as e:  # pragma: no cover
            log("NVML unavailable:", e)
            return
        self.nv = pynvml
        self.sample_s = []
        self.h = pynvml.nvmlDeviceGetHandleByIndex(self.device)
        self.stop_ev = threading.Event()
        self.kick_ev = threading.Event() if kicked else None
        bits = {"hw_slowdown": pynvml.nvmlClocksEventReasonHwSlowdown,
                "hw_thermal_slowdown": pynvml.nvmlClocksEventReasonHwThermalSlowdown,
                "sw_thermal_slowdown": pynvml.nvmlClocksEventReasonSwThermalSlowdown,
                "sw_power_cap": pynvml.nvmlClocksEventReasonSwPowerCap}

        mx = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)   # once: this query takes ms

        def run():
            while not self.stop_ev.is_set():
                if self.kick_ev is not None:
                    if not self.kick_ev.wait(0.05):
                        continue
                    self.kick_ev.clear()
                    time.sleep(0.01)          # inside the PageRank call
                t0 = time.perf_counter()
                sm = pynvml.nvmlDeviceGetClockInfo(self.h, pynvml.NVML_CLOCK_SM)
                r = pynvml.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                self.sample_s.append(time.perf_counter() - t0)
                act = ["Active" if r & b else "Not Active" for b in bits.values()]
                self.lines.append(", ".join([str(sm), str(mx), "0", hex(r)] + act))
                if self.kick_ev is None:
                    self.stop_ev.wait(0.2)
        self.t = threading.Thread(target=run, daemon=True)
        self.t.start()
        self.proc = "nvml"

    def stop(self):
        if not self.proc:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["clock sampling off"]}
        if self.proc == "nvml":
            self.stop_ev.set()
            self.t.join(timeout=5)
        else:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 8:
                continue
            try:
                sm.append(float(f[0]))
                mx.append(float(f[1]))
            except ValueError:
                continue
            for nm, v in zip(names, f[4:8]):
                if v.lower() == "active":
                    reasons.add(nm)
        out = {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(mx) if mx else None,
               "reasons": sorted(reasons), "samples": len(sm)}
        if getattr(self, "sample_s", None):
            out["nvml_query_ms_max"] = round(1e3 * max(self.sample_s), 3)
        return out


# --------------------------------------------------------------------- reference arm ---

def run_reference(args, rank):
    """The reference arm (this tier has no installable reference): the oracle, as it stands,
    on every host core (OpenMP build, level-synchronous BFS -- the metric's algorithm) on a
    bounded RMAT-24 sample of the workload, one BFS per step (rank 0 only)."""
    if rank != 0:
        return
    import inputs
    import oracle
    scale = args.ref_scale
    log(f"[reference] generating RMAT-{scale} sample")
    g = inputs.rmat(scale)
    times, edges = [], 0
    deg = np.diff(g.row_ptr).astype(np.int64)
    for i in range(args.warmup + args.steps):
        t0 = time.perf_counter()
        lv = oracle.bfs_levelsync(g.row_ptr, g.col, 0, omp=True)
        dt = time.perf_counter() - t0
        if i >= args.warmup:
            times.append(dt)
        edges = int(deg[lv != oracle.UNREACHED].sum())
    t = float(np.sum(times))
    gteps = edges * len(times) / t / 1e9
    threads = oracle.num_threads(omp=True)
    line = {"impl": "reference", "metric": METRIC, "value": gteps, "unit": "GTEPS", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * t / len(times),
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "u32",
            "data": "synthetic",
            "config": {"workload": f"rmat{args.scale}_bfs_pr_sssp_wcc", "scale": args.scale, "src": 0,
                       "sample": f"reference arm: oracle BFS (the metric's algorithm) on the RMAT-{scale} sample",
                       "sample_scale": scale},
            "cpu_baseline": {"value": gteps, "unit": "GTEPS", "cores": threads, "kind": "oracle", "host": host_info(),
                             "sample": f"oracle level-synchronous BFS (OpenMP build, {threads} threads) from vertex 0 "
                                       f"on RMAT-{scale} (same generator as RMAT-{args.scale}, "
                                       f"1/{2 ** (args.scale - scale)} of its edges), per step"},
            "e2e": {"value": gteps, "unit": "GTEPS", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ----------------------------------------------------------------------------- GPU arm ---

def host_info():
    """nproc and the lscpu model / sockets / cores of the host the oracle runs on."""
    info = {"nproc": os.cpu_count()}
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for ln in out.splitlines():
            k, _, v = ln.partition(":")
            k = k.strip()
            if k in ("Model name", "Socket(s)", "Core(s) per socket", "Thread(s) per core"):
                info[k] = v.strip()
    except Exception:  # pragma: no cover
        pass
    return info


def oracle_bfs_all_cores(g, src):
    """The oracle's level-synchronous BFS (OpenMP build, every host core) on the bench
    graph itself: the all-core CPU baseline and the level array B_BFS is computed from."""
    import oracle
    t0 = time.perf_counter()
    lv = oracle.bfs_levelsync(g.row_ptr, g.col, src, omp=True)
    return lv, time.perf_counter() - t0


def cpu_baseline(args, have_full=None, full_t=None, full_edges=None):
    """the oracle as it stands on the GPU box's host cores -- (1) every core
    (OpenMP build) on the bench workload itself (BFS, the metric's algorithm), (2) one core
    (plain build) on an RMAT-24 sample, and the PageRank iteration time of the OpenMP build
    on that sample (t(2 iterations) - t(1 iteration): the transpose is excluded)."""
    import inputs
    import oracle
    scale = args.ref_scale
    g = inputs.rmat(scale)
    deg = np.diff(g.row_ptr).astype(np.int64)
    t0 = time.perf_counter()
    lv = oracle.bfs(g.row_ptr, g.col, 0)
    t_bfs = time.perf_counter() - t0
    edges = int(deg[lv != oracle.UNREACHED].sum())
    t0 = time.perf_counter()
    oracle.pagerank(g.row_ptr, g.col, 1, 0.85, omp=True)
    t1 = time.perf_counter() - t0
    t0 = time.perf_counter()
    oracle.pagerank(g.row_ptr, g.col, 2, 0.85, omp=True)
    t2 = time.perf_counter() - t0
    threads = oracle.num_threads(omp=True)
    out = {"unit": "GTEPS", "kind": "oracle", "host": host_info(),
           "one_core": {"value": edges / t_bfs / 1e9, "cores": 1, "bfs_s": t_bfs,
                        "sample": f"oracle FIFO-queue BFS from vertex 0 on RMAT-{scale} (same generator, "
                                  f"1/{2 ** (args.scale - scale)} of the RMAT-{args.scale} edges), plain build"},
           "pagerank_s_per_iter_sample": max(t2 - t1, 0.0), "pagerank_sample": f"RMAT-{scale}, OpenMP build, "
           f"{threads} threads, t(2 iterations) - t(1 iteration)"}
    if have_full:
        out.update({"value": full_edges / full_t / 1e9, "cores": threads, "bfs_s": full_t,
                    "sample": f"oracle level-synchronous BFS (OpenMP build, {threads} threads = every host core) "
                              f"on the bench graph itself, from the bench source, once"})
    else:
        out.update({"value": out["one_core"]["value"], "cores": 1, "sample": out["one_core"]["sample"]})
    return out


def bfs_algorithmic_bytes(lv_caller, row_ptr, gr):
    """B_BFS of SURVEY 8(d), from the oracle's level array and the page directory:
    sum over levels of the frontier-bitmap bits of each active page (nslots / 8 bytes;
    LP continuation pages, 1 bit each, are not counted) + per reached vertex its slot
    offset, ADJLIST_SZ and adjacency (4 + 4 + 4 deg; the slot's VID is implied by its
    position) + a 4-byte visited test per traversed edge + a 4-byte LV write per reached
    vertex.  Independent of the GPU's timing."""
    import oracle
    reached = lv_caller != oracle.UNREACHED
    deg = np.diff(row_ptr).astype(np.int64)
    edges = int(deg[reached].sum())
    nr = int(reached.sum())
    d = gr.directory()
    internal = gr.order()
    ids = internal[reached].astype(np.int64)
    page = np.searchsorted(d["start_vid"].astype(np.int64), ids, side="right") - 1
    lev = lv_caller[reached].astype(np.int64)
    key = np.unique(lev * (1 << 32) + page)
    frontier_bits = float(d["nslots"][key & 0xFFFFFFFF].astype(np.int64).sum()) / 8.0
    b = frontier_bits + 12.0 * nr + 4.0 * edges + 4.0 * edges + 4.0 * nr
    return b, {"frontier_bitmap": frontier_bits, "slot_len_adj": 12.0 * nr + 4.0 * edges,
               "visited_tests": 4.0 * edges, "lv_writes": 4.0 * nr, "edges": edges, "reached": nr,
               "active_page_levels": int(key.size)}


def h2d_peak_gbs(nbytes=256 << 20, reps=10):
    """Pinned host -> device copy bandwidth in this process (cudaMemcpyAsync via torch), best of reps."""
    import torch
    h = torch.empty(nbytes, dtype=torch.uint8, pin_memory=True)
    d = torch.empty(nbytes, dtype=torch.uint8, device="cuda")
    best = 0.0
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        d.copy_(h, non_blocking=True)
        e1.record()
        torch.cuda.synchronize()
        best = max(best, nbytes / (e0.elapsed_time(e1) * 1e-3) / 1e9)
    return best


def make_graph(args, rank, world, dist):
    """The workload graph.  With N > 1 ranks on one node, rank 0 draws it once
    and shares the CSR through /dev/shm (each rank then builds its own pages)."""
    import inputs
    gen = (lambda: inputs.rmat(args.scale)) if args.workload == "rmat" else inputs.twitter_like
    if world == 1:
        return gen()
    obj = [None]
    if rank == 0:
        g = gen()
        # /dev/shm when it has room for the CSR (a container's default is 64 MB), else the temp dir
        need = g.row_ptr.nbytes + g.col.nbytes + (1 << 30)
        base = "/dev/shm"
        try:
            if shutil.disk_usage(base).free < need:
                base = tempfile.gettempdir()
        except OSError:
            base = tempfile.gettempdir()
        tag = os.path.join(base, f"gts_bench_{args.workload}_{args.scale}_{os.environ.get('MASTER_PORT', '0')}")
        np.save(tag + "_rp.npy", g.row_ptr)
        np.save(tag + "_col.npy", g.col)
        obj = [tag]
    dist.broadcast_object_list(obj, src=0)
    args._shared_tag = obj[0]
    if rank != 0:
        g = inputs.CSR(np.load(obj[0] + "_rp.npy", mmap_mode="r"), np.load(obj[0] + "_col.npy", mmap_mode="r"))
    return g


def drop_shared_graph(args, rank, world, dist):
    if world > 1:
        dist.barrier()
        if rank == 0:
            for suf in ("_rp.npy", "_col.npy"):
                try:
                    os.remove(args._shared_tag + suf)
                except OSError:
                    pass


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="gts", choices=["gts", "reference"])
    ap.add_argument("--scale", type=int, default=27)
    ap.add_argument("--workload", default="rmat", choices=["rmat", "twitter"],
                    help="rmat: RMAT-<scale> (configs[2]); twitter: Twitter-shaped (configs[1])")
    ap.add_argument("--ref-scale", type=int, default=None)
    ap.add_argument("--page-bytes", type=int, default=1 << 20)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-streamed", action="store_true", help="skip the streamed-topology leg (a3)")
    ap.add_argument("--strategy", default="P", choices=["P", "S", "S_BCAST"],
                    help="multi-GPU strategy for N > 1 (SURVEY 8(e)); P = the default scaling run")
    ap.add_argument("--algos", default="bfs,pr,sssp,wcc")
    ap.add_argument("--order", dest="order", action="store_true", default=True,
                    help="build pages with GTS_BUILD_DEGREE_ORDER (default)")
    ap.add_argument("--no-order", dest="order", action="store_false")
    args = ap.parse_args()
    if args.ref_scale is None:
        args.ref_scale = min(args.scale, 24)
    args.warmup = max(args.warmup, 3) if args.impl == "gts" else args.warmup

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if args.gpus > 1 and world != args.gpus:
        sys.exit(f"--gpus {args.gpus} must be launched with torchrun --nproc-per-node {args.gpus}")

    if args.impl == "reference":
        run_reference(args, rank)
        return

    import torch
    import torch.distributed as dist

    import inputs
    import paper_conf_sigmod_0002apsk16_b200 as G

    torch.cuda.set_device(local_rank)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local_rank))
        os.environ.setdefault("OMP_NUM_THREADS", str(max(1, os.cpu_count() // world)))
    algos = args.algos.split(",")

    t0 = time.time()
    g = make_graph(args, rank, world, dist)
    n, m = g.n, g.m
    src = 0 if args.workload == "rmat" else int(np.argmax(np.diff(g.row_ptr)))
    wname = f"rmat{args.scale}" if args.workload == "rmat" else "twitter_shaped"
    log(f"[rank {rank}] {wname} generated n={n} m={m} in {time.time() - t0:.1f}s")
    # the oracle on every host core, on this very graph: the all-core CPU baseline and the
    # level array the algorithmic BFS bytes (roofline_bfs) are computed from
    lv_oracle = t_oracle = None
    if rank == 0 and not args.no_cpu_baseline and "bfs" in algos:
        lv_oracle, t_oracle = oracle_bfs_all_cores(g, src)
        log(f"[rank 0] oracle BFS on all host cores: {t_oracle:.2f}s")
    t0 = time.time()
    strat = {"P": G.GTS_STRATEGY_P, "S": G.GTS_STRATEGY_S, "S_BCAST": G.GTS_STRATEGY_S_BCAST}[args.strategy]
    # N > 1: every rank builds and pins only the pages it processes (GTS_BUILD_OWNER_FILTER),
    # so host page bytes per rank are ~T_topo / N
    own = (rank, world, strat) if world > 1 else None
    gr = G.gts_build_pages(g.row_ptr, g.col, page_bytes=args.page_bytes, order=args.order, owner=own)
    grs = None
    if "wcc" in algos and world > 1 and strat == G.GTS_STRATEGY_S:   # routed WCC: symmetrised pages
        grs = G.gts_build_pages(g.row_ptr, g.col, page_bytes=args.page_bytes, order=args.order, owner=own,
                                symmetric=True)
    grw = None
    if "sssp" in algos:
        w = inputs.edge_weights(g)
        grw = G.gts_build_pages(g.row_ptr, g.col, w, page_bytes=args.page_bytes, order=args.order, owner=own)
        del w
    gst = gr.stats()
    log(f"[rank {rank}] pages built in {time.time() - t0:.1f}s: {gst}")
    B_bfs = bfs_parts = edges_oracle = None
    if lv_oracle is not None:
        B_bfs, bfs_parts = bfs_algorithmic_bytes(lv_oracle, g.row_ptr, gr)
        edges_oracle = bfs_parts["edges"]
        del lv_oracle
    del g
    drop_shared_graph(args, rank, world, dist)

    uid = None
    if world > 1:
        obj = [G.gts_get_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        uid = obj[0]
    ctx = G.gts_context_create(local_rank, rank, world, uid)
    stream = torch.cuda.current_stream()
    ctx.set_stream(stream.cuda_stream)

    lv = torch.empty(n, dtype=torch.int32, device="cuda")
    pr = torch.empty(n, dtype=torch.float32, device="cuda")
    ds = torch.empty(n, dtype=torch.int32, device="cuda")
    lab = torch.empty(n, dtype=torch.int32, device="cuda")

    def step(record):
        evs = {}
        res = {}
        for a in algos:
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            if a == "bfs":
                _, st = G.gts_bfs(ctx, gr, src, out=lv, timing=True, strategy=strat)
            elif a == "pr":
                if sampler is not None:
                    sampler.kick()
                _, st = G.gts_pagerank(ctx, gr, 10, 0.85, out=pr, timing=True, strategy=strat)
            elif a == "sssp":
                _, st = G.gts_sssp(ctx, grw, src, out=ds, timing=True, strategy=strat)
            else:
                _, st = G.gts_wcc(ctx, grs if grs is not None else gr, out=lab, timing=True, strategy=strat)
            e1.record(stream)
            evs[a] = (e0, e1)
            res[a] = st
        torch.cuda.synchronize()
        if record is not None:
            for a in algos:
                record.setdefault(a, []).append((evs[a][0].elapsed_time(evs[a][1]) * 1e-3, res[a]))

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    sampler = None
    for i in range(args.warmup):
        step(None)
        log(f"[rank {rank}] warmup {i} done")
    sampler = ClockSampler(local_rank)
    sampler.start()
    if "pr" not in algos:             # no PageRank call to sample inside: sample at each step start
        _step = step

        def step(record):
            sampler.kick()
            _step(record)
    rec = {}
    # no cyclic-GC pause inside the timed region (a collection between two calls would idle
    # the GPU while the host is stopped)
    gc.collect()
    gc.disable()
    barrier()
    t_start = torch.cuda.Event(enable_timing=True)
    t_end = torch.cuda.Event(enable_timing=True)
    t_start.record(stream)
    for _ in range(args.steps):
        step(rec)
    t_end.record(stream)
    barrier()
    gc.enable()
    clocks = sampler.stop()
    total_s = t_start.elapsed_time(t_end) * 1e-3

    def maxred(x):
        if world == 1:
            return x
        t = torch.tensor([x], dtype=torch.float64, device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    def sumred(x):
        if world == 1:
            return x
        t = torch.tensor([x], dtype=torch.float64, device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.SUM)
        return float(t.item())

    total_s = maxred(total_s)
    out = {}
    for a in algos:
        out[a] = {"s": maxred(sum(t for t, _ in rec[a])),
                  "main_s": maxred(sum(st["main_kernel_s"] for _, st in rec[a])),
                  "main_launches": sum(st["main_kernel_launches"] for _, st in rec[a]),
                  "launches": sum(st["launches"] for _, st in rec[a]),
                  "edges": sumred(float(sum(st["edges_traversed"] for _, st in rec[a]))),
                  "iters": rec[a][-1][1]["levels_or_iters"],
                  "merge_s": maxred(sum(st["merge_s"] for _, st in rec[a]))}
    K = args.steps
    bfs_gteps = out["bfs"]["edges"] / out["bfs"]["s"] / 1e9 if "bfs" in algos else None
    pr_s_iter = out["pr"]["s"] / (10 * K) if "pr" in algos else None

    # roofline for the dominant kernel (largest share of the step among the main kernels)
    peak, peak_src = measured_peaks()
    B_pr_scatter = 12 * m + 16 * n          # topology 4m+12n, x 4n, acc RMW 8m
    cand = {}
    if "pr" in algos:
        cand["pr_scatter_kernel"] = (out["pr"]["main_s"], out["pr"]["main_launches"], B_pr_scatter / world)
    if "wcc" in algos:
        cand["wcc_sweep_kernel"] = (out["wcc"]["main_s"], out["wcc"]["main_launches"], (4 * m + 12 * n + 8 * m) / world)
    if "bfs" in algos:
        eb = out["bfs"]["edges"] / K
        cand["bfs_expand_kernel"] = (out["bfs"]["main_s"], out["bfs"]["main_launches"],
                                     (4 * eb + 12 * n + 4 * eb) / max(1, out["bfs"]["main_launches"] / K) / world)
    dom = max(cand, key=lambda k: cand[k][0]) if cand else None
    roof = None
    if dom:
        ks, kl, bytes_per_launch = cand[dom]
        avg = ks / max(1, kl)
        ach = bytes_per_launch / avg / 1e9 if avg > 0 else 0.0
        traffic, tj, tw = None, {}, {}
        tp = os.path.join(ROOT, "profiles", "traffic.json")
        if os.path.exists(tp):        # ncu --set full captures, per workload (profiles/)
            tj = json.load(open(tp))
            tw = tj.get(f"{wname}_bfs_pr_sssp_wcc", {}) if world == 1 else {}
            traffic = tw.get(dom)
        roof = {"bound": "hbm", "kernel": dom, "achieved": ach, "peak": peak, "unit": "GB/s", "frac": ach / peak,
                "traffic": traffic, "algorithmic_bytes_per_launch": bytes_per_launch, "avg_launch_s": avg,
                "share_of_step": ks / total_s if total_s else None, "peak_source": peak_src}
        red = tw.get(dom + "_lts_red_sectors")
        if red and avg > 0:   # the scatter's real ceiling: L2 atomic throughput
            roof["l2_red"] = {"ops_per_launch_ncu": red, "achieved_gops": red / avg / 1e9,
                              "ceiling_gops": tj.get("l2_red_ceiling_gops"),
                              "frac": red / avg / 1e9 / tj.get("l2_red_ceiling_gops", 1.0),
                              "ceiling_source": tj.get("_l2_red_source")}

    roof_bfs = None
    if B_bfs is not None and out["bfs"]["main_s"] > 0:
        t_call = out["bfs"]["main_s"] / K          # the BFS kernels of one call (all levels)
        roof_bfs = {"bound": "hbm", "kernel": "bfs_expand_kernel (+ finish / page-set kernels)",
                    "achieved": B_bfs / t_call / 1e9, "peak": peak, "unit": "GB/s", "frac": B_bfs / t_call / 1e9 / peak,
                    "algorithmic_bytes_per_call": B_bfs, "parts": bfs_parts, "kernel_s_per_call": t_call,
                    "peak_source": peak_src,
                    "what": "B_BFS of SURVEY 8(d) from the oracle's levels and the page directory / the BFS "
                            "kernels' CUDA-event time per call"}

    # end-to-end through the public API with host buffers (pages re-uploaded from pinned host memory)
    e2e = None
    if not args.no_e2e and "bfs" in algos:
        hl = torch.empty(n, dtype=torch.int32, pin_memory=True)      # pinned host result buffers
        hp = torch.empty(n, dtype=torch.float32, pin_memory=True)
        tb, tp_ = [], []
        for _ in range(max(1, min(K, 5))):
            ctx.evict(gr)
            barrier()
            t0 = time.perf_counter()
            _, st = G.gts_bfs(ctx, gr, src, out=hl, strategy=strat)
            tb.append(maxred(time.perf_counter() - t0))
            ctx.evict(gr)
            barrier()
            t0 = time.perf_counter()
            G.gts_pagerank(ctx, gr, 10, 0.85, out=hp, strategy=strat)
            tp_.append(maxred(time.perf_counter() - t0))
        e2e = {"value": out["bfs"]["edges"] / K / float(np.median(tb)) / 1e9, "unit": "GTEPS",
               "h2d_bytes_per_step": int(gst["topo_bytes"] / world), "d2h_bytes_per_step": 4 * n,
               "what": "gts_bfs on an evicted context with a host output: H2D of this rank's pinned pages + BFS + "
                       "D2H of the level array, wall clock, median",
               "pagerank_s_per_iter": float(np.median(tp_)) / 10}

    # streamed topology (a3): pages from pinned host memory through the ring, after the timed region
    streamed = None
    if not args.no_streamed and world == 1 and "pr" in algos and "bfs" in algos:
        peak_h2d = h2d_peak_gbs()
        ctx.evict(gr)
        # one untimed streamed iteration first: the ring and its events are allocated on
        # the first streamed call (a cold 2-iteration measurement read 0.68 of the link)
        G.gts_pagerank(ctx, gr, 1, 0.85, out=pr, residency=G.GTS_STREAMED)
        torch.cuda.synchronize()
        SPI = 3
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        _, sp = G.gts_pagerank(ctx, gr, SPI, 0.85, out=pr, residency=G.GTS_STREAMED, timing=True)
        e1.record(stream)
        torch.cuda.synchronize()
        t_pr = e0.elapsed_time(e1) * 1e-3 / SPI
        e0.record(stream)
        _, sb = G.gts_bfs(ctx, gr, src, out=lv, residency=G.GTS_STREAMED, timing=True)
        e1.record(stream)
        torch.cuda.synchronize()
        t_bfs = e0.elapsed_time(e1) * 1e-3
        link_pr = sp["h2d_bytes"] / SPI / t_pr / 1e9
        link_bfs = sb["h2d_bytes"] / t_bfs / 1e9
        streamed = {"pagerank_s_per_iter": t_pr, "bfs_gteps": sb["edges_traversed"] / t_bfs / 1e9, "bfs_s": t_bfs,
                    "h2d_bytes_per_pr_iter": sp["h2d_bytes"] / SPI, "h2d_bytes_bfs": sb["h2d_bytes"],
                    "link_gbs_pr": link_pr, "link_gbs_bfs": link_bfs, "h2d_peak_gbs": peak_h2d,
                    "link_frac": link_pr / peak_h2d, "link_frac_bfs": link_bfs / peak_h2d,
                    "what": "GTS_STREAMED (forced): topology pages copied from pinned host memory into a 4 x 64 MiB "
                            "device ring per iteration / level, kernels overlapped; RA/WA resident; PageRank: 3 "
                            "iterations after an untimed one; CUDA events "
                            "on the call stream; peak = pinned H2D of 256 MiB in this process, best of 10"}

    cpu = None
    if rank == 0 and not args.no_cpu_baseline:
        try:
            cpu = cpu_baseline(args, t_oracle is not None, t_oracle, edges_oracle)
        except Exception as e:  # pragma: no cover
            cpu = {"error": str(e)}

    if rank == 0:
        line = {"metric": METRIC, "value": bfs_gteps, "unit": "GTEPS", "n_gpus": world, "steps": K,
                "warmup": args.warmup, "ms_per_step": 1e3 * total_s / K, "higher_is_better": True,
                "scaling": "strong", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
                "config": {"workload": f"{wname}_bfs_pr_sssp_wcc", "scale": args.scale if args.workload == "rmat" else None,
                           "n": n, "m": m, "edge_factor": 16 if args.workload == "rmat" else None,
                           "abc": [0.57, 0.19, 0.19] if args.workload == "rmat" else None,
                           "seed": args.scale if args.workload == "rmat" else inputs.TWITTER_SEED, "src": src,
                           "page_bytes": args.page_bytes, "num_pages": gst["num_pages"], "n_lp": gst["n_lp"],
                           "vertex_order": "in-degree (GTS_BUILD_DEGREE_ORDER)" if args.order else "VID",
                           "topo_bytes": gst["topo_bytes"], "residency": "resident",
                           "strategy": args.strategy if world > 1 else "single",
                           "parallelism": f"strategy-{args.strategy} x{world}",
                           "host_page_bytes_per_rank": gst["host_page_bytes"],
                           "l2": "inputs larger than L2 (topology %.1f GB vs 126 MB L2), no flush" %
                                 (gst["topo_bytes"] / 1e9),
                           "step": "+".join(algos)},
                "pagerank_s_per_iter": pr_s_iter, "pagerank_dtype": "f32",
                "bfs_levels": out.get("bfs", {}).get("iters"),
                "sssp_s": out["sssp"]["s"] / K if "sssp" in algos else None,
                "sssp_rounds": out.get("sssp", {}).get("iters"),
                "wcc_s": out["wcc"]["s"] / K if "wcc" in algos else None,
                "wcc_sweeps": out.get("wcc", {}).get("iters"),
                "kernel_s_per_step": {a: out[a]["main_s"] / K for a in algos},
                "call_ms_each_step": {a: [round(1e3 * t, 3) for t, _ in rec[a]] for a in algos},
                "merge_s_per_step": {a: out[a]["merge_s"] / K for a in algos},
                "roofline": roof, "roofline_bfs": roof_bfs, "streamed": streamed,
                "cpu_baseline": cpu, "e2e": e2e, "clocks": clocks,
                "gpu_launches": int(sum(out[a]["launches"] for a in algos))}
        print(json.dumps(line), flush=True)
    ctx.free()
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
