"""GTS cost models (section 5, Eq 1 P:446-474 and Eq 2)
evaluated with constants measured on B200, against the measured streamed runs
(SURVEY 8(f) NEXT #3).

Eq 1 (PageRank-like, one iteration, N GPUs):
    T = 2 sz(WA)/c1 + (sz(RA) + sz(SP) + sz(LP)) / (c2 N) + t_call((S+L)/N) + t_kernel(SP1 + LP1) + t_sync(N)
Eq 2 (BFS-like):
    T = 2 sz(WA)/c1 + sum_l [ (sz(RA_l) + sz(SP_l) + sz(LP_l)) / (c2 N d_skew) (1 - r_hit) + t_call((S_l+L_l)/(N d_skew)) ]

B200 design differences that zero some terms: WA and RA stay resident in HBM
(no chunk copy, RA not streamed), and pages move in batches of B (t_call per
batch, not per page).  c2 = the measured pinned H2D rate; t_call per batch is
fitted from the ring/batch sweep (the batch-of-1 runs are launch bound).

    python tools/cost_model.py profiles/r01_stream_rmat27.json profiles/r01_stream_sweep_rmat27.json
"""
import json
import sys


def main(stream_path, sweep_path):
    st = json.load(open(stream_path))
    sw = json.load(open(sweep_path))
    c2 = st["h2d_peak_gbs"] * 1e9
    topo = st["topo_bytes"]
    pages = st["num_pages"]
    page = topo / pages
    # t_call + t_kernel per batch: from the batch-of-1 sweep (copy of one page + one launch per page)
    one = min(r["s_per_iter"] for r in sw["sweep"] if r["batch_pages"] == 1)
    t_batch = one / pages - page / c2
    rows = []
    for r in sw["sweep"]:
        B = r["batch_pages"]
        batches = -(-pages // B)
        copy_b = B * page / c2                 # a batch's copy; its kernel runs B pages on B CTAs in parallel
        pred = batches * (copy_b + t_batch) if r["ring"] == 1 else batches * max(copy_b, t_batch) + t_batch
        rows.append((r["ring"], B, pred, r["s_per_iter"]))
    print(f"c2 = {c2 / 1e9:.1f} GB/s (measured pinned H2D), topology {topo / 1e9:.2f} GB in {pages} pages, "
          f"t_call+t_kernel per batch = {t_batch * 1e6:.0f} us (fitted from the batch-of-1 runs)")
    print("per iteration: ring 1 = batches * (copy + kernel); ring >= 2 = batches * max(copy, kernel) + kernel")
    print("Eq 1, PageRank iteration, N = 1:")
    print(f"  {'ring':>4} {'batch':>5} {'predicted_s':>11} {'measured_s':>10} {'ratio':>6}")
    for ring, B, p, m in rows:
        print(f"  {ring:4d} {B:5d} {p:11.3f} {m:10.3f} {m / p:6.2f}")
    pr = st["pagerank"]
    print(f"  default ring/batch: predicted {topo / c2:.3f} s (link term), measured {pr['s_per_iter']:.3f} s")
    bfs = st["bfs"]
    pred = bfs["h2d_bytes"] / c2
    print(f"Eq 2, BFS, N = 1, r_hit = 0 (no cache), d_skew = 1: sum_l sz(SP_l)/c2 = {pred:.3f} s, "
          f"measured {bfs['s']:.3f} s ({bfs['pages_processed']} page visits over {bfs['levels']} levels)")


if __name__ == "__main__":
    main(*sys.argv[1:3])
