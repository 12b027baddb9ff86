"""N > 1 host logic on CPU: world_size-2 (and 3) process groups over gloo.

Each rank takes the pages libgts assigns it (gts_partition_pages: Strategy-P
h(j) = j mod N; Strategy-S contiguous WA ranges), reads
ONLY those pages (through the oracle's page reader), computes its partial
sweep, and merges with the same collective algebra libgts issues over NCCL:

* PageRank P: all_reduce(sum) of the edge-term accumulator and of the dangling
  mass D, teleport applied once after the merge (R17);  S: the accumulator is
  reduced and each rank finishes only its own VID range, then ranges are
  gathered.
* BFS: all_gather of the next-frontier bitmaps + OR (NCCL has no bitwise OR).
* WCC / SSSP: all_reduce(min).

Results must equal the single-process oracle (bit-exact for BFS/WCC/SSSP,
1e-12 for the fp64 PageRank model).
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _my_part(G, oracle, gr, g, pb, strategy, world, rank):
    owner, vrange = G.gts_partition_pages(gr, strategy, world)
    d = gr.directory()
    pages = gr.pages().reshape(-1, pb)
    mine = np.nonzero(owner == rank)[0]
    rp, col, w = oracle.decode_pages(pages[mine].reshape(-1), pb, g.n, g.m, weighted=bool(gr.stats()["weighted"]))
    verts = np.zeros(g.n, dtype=bool)          # vertices whose records live in my pages
    for p in mine:
        verts[d["start_vid"][p]:d["start_vid"][p] + d["nslots"][p]] = True
    src = np.repeat(np.arange(g.n), np.diff(rp).astype(np.int64))
    return owner, vrange, verts, src, col.astype(np.int64), w


def _worker(rank, world, port, out):
    import sys
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import inputs
    import oracle
    import paper_conf_sigmod_0002apsk16_b200 as G
    res = {}
    try:
        g = inputs.rmat(12).with_weights()
        pb = 4096
        gr = G.gts_build_pages(g.row_ptr, g.col, page_bytes=pb)
        grw = G.gts_build_pages(g.row_ptr, g.col, g.weights, page_bytes=2 * pb)
        outdeg = np.diff(g.row_ptr).astype(np.float64)
        n, d = g.n, 0.85
        for strategy in (G.GTS_STRATEGY_P, G.GTS_STRATEGY_S):
            owner, vrange, verts, src, dst, _ = _my_part(G, oracle, gr, g, pb, strategy, world, rank)
            lo, hi = int(vrange[rank]), int(vrange[rank + 1])
            if strategy == G.GTS_STRATEGY_S:   # S: every source of my pages is in my WA range
                assert np.all((src >= lo) & (src < hi))
                assert np.all(np.nonzero(verts)[0] >= lo) and np.all(np.nonzero(verts)[0] < hi)
            # ---- PageRank
            x = np.full(n, 1.0 / n)
            for _ in range(10):
                acc = np.zeros(n)
                np.add.at(acc, dst, d * x[src] / outdeg[src])
                D = np.array([x[verts & (outdeg == 0)].sum()])
                ta, tD = torch.from_numpy(acc), torch.from_numpy(D)
                dist.all_reduce(ta)
                dist.all_reduce(tD)
                newx = (1 - d) / n + d * tD.item() / n + ta.numpy()
                if strategy == G.GTS_STRATEGY_S:
                    part = np.zeros(n)
                    part[lo:hi] = newx[lo:hi]            # finish only my range ...
                    tp = torch.from_numpy(part)
                    dist.all_reduce(tp)                  # ... then gather the ranges
                    newx = tp.numpy()
                x = newx
            res[("pr", strategy)] = float(np.max(np.abs(x - oracle.pagerank(g.row_ptr, g.col, 10, d))))
            # ---- BFS
            lv = np.full(n, oracle.UNREACHED, dtype=np.uint32)
            lv[0] = 0
            front = np.zeros(n, dtype=bool)
            front[0] = True
            level = 0
            while front.any():
                sel = front[src]
                nxt = np.zeros(n, dtype=bool)
                nxt[dst[sel]] = True
                nxt &= lv == oracle.UNREACHED
                bits = torch.from_numpy(np.packbits(nxt))
                gathered = [torch.zeros_like(bits) for _ in range(world)]
                dist.all_gather(gathered, bits)
                merged = np.bitwise_or.reduce(np.stack([t.numpy() for t in gathered]), axis=0)
                front = np.unpackbits(merged)[:n].astype(bool)
                level += 1
                lv[front] = level
            res[("bfs", strategy)] = bool(np.array_equal(lv, oracle.bfs(g.row_ptr, g.col, 0)))
            # ---- WCC (min-label propagation + all_reduce(min) per sweep)
            lab = np.arange(n, dtype=np.int64)
            while True:
                before = lab.copy()
                m_ = np.minimum(lab[src], lab[dst])
                np.minimum.at(lab, dst, m_)
                np.minimum.at(lab, src, m_)
                t = torch.from_numpy(lab)
                dist.all_reduce(t, op=dist.ReduceOp.MIN)
                lab = t.numpy().copy()
                lab = lab[lab]
                ch = torch.tensor([int(np.any(lab != before))])
                dist.all_reduce(ch, op=dist.ReduceOp.MAX)
                if ch.item() == 0:
                    break
            res[("wcc", strategy)] = bool(np.array_equal(lab.astype(np.uint32), oracle.wcc(g.row_ptr, g.col)))
            # ---- SSSP (frontier Bellman-Ford + all_reduce(min) per round)
            _, _, vw, sw, dw, ww = _my_part(G, oracle, grw, g, 2 * pb, strategy, world, rank)
            INF = np.iinfo(np.int64).max // 4
            dd = np.full(n, INF, dtype=np.int64)
            dd[0] = 0
            front = np.zeros(n, dtype=bool)
            front[0] = True
            while True:
                sel = front[sw]
                cand = dd[sw[sel]] + ww[sel].astype(np.int64)
                new = dd.copy()
                np.minimum.at(new, dw[sel], cand)
                t = torch.from_numpy(new)
                dist.all_reduce(t, op=dist.ReduceOp.MIN)
                new = t.numpy()
                front = new < dd
                dd = new.copy()
                if not front.any():
                    break
            want = oracle.sssp(g.row_ptr, g.col, g.weights, 0).astype(np.int64)
            got = np.where(dd >= INF, oracle.UNREACHED, dd)
            res[("sssp", strategy)] = bool(np.array_equal(got, want))
    except Exception as e:  # pragma: no cover
        res["error"] = repr(e)
    out[rank] = res
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_gloo_strategies(world):
    ctx = mp.get_context("spawn")
    mgr = ctx.Manager()
    out = mgr.dict()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, out)) for r in range(world)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(300)
    assert all(p.exitcode == 0 for p in procs)
    for r in range(world):
        res = out[r]
        assert "error" not in res, res
        for strategy in (0, 1):
            assert res[("pr", strategy)] <= 1e-12, res
            assert res[("bfs", strategy)], res
            assert res[("wcc", strategy)], res
            assert res[("sssp", strategy)], res


def _owner_worker(rank, world, port, strategy, out):
    import sys
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import inputs
    import paper_conf_sigmod_0002apsk16_b200 as G
    try:
        g = inputs.rmat(14)
        pb = 8192
        # each process builds and holds only its own pages (libgts GTS_BUILD_OWNER_FILTER)
        gr = G.gts_build_pages(g.row_ptr, g.col, page_bytes=pb, order=True, owner=(rank, world, strategy))
        st = gr.stats()
        owner, vr = G.gts_partition_pages(gr, strategy, world)
        mine = np.nonzero(owner == rank)[0]
        got = [None] * world
        dist.all_gather_object(got, (mine, gr.pages(), st["host_page_bytes"]))
        if rank == 0:
            full = G.gts_build_pages(g.row_ptr, g.col, page_bytes=pb, order=True)
            fp = full.pages().reshape(-1, pb)
            seen = np.zeros(fp.shape[0], np.int64)
            for ids, pages, hb in got:
                assert hb == len(ids) * pb
                assert np.array_equal(pages.reshape(-1, pb), fp[ids])
                seen[ids] += 1
            out.put(("ok", bool(np.all(seen == 1)), [hb for _, _, hb in got], full.stats()["topo_bytes"]))
    except Exception as e:  # pragma: no cover
        out.put(("err", repr(e)))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
@pytest.mark.parametrize("strategy", [0, 1])
def test_gloo_owner_filtered_builds(world, strategy):
    """One process per rank (gloo): every rank builds only its pages through libgts;
    together they hold every page exactly once, byte-identical to a full build, with
    host page bytes ~T_topo / N per rank (the multi-GPU memory plan)."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_owner_worker, args=(r, world, port, strategy, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = q.get(timeout=300)
    for p in procs:
        p.join(timeout=120)
    assert res[0] == "ok", res
    _, partition_ok, host_bytes, topo = res
    assert partition_ok
    assert sum(host_bytes) == topo
    assert max(host_bytes) <= topo / world * 1.2 + 16384
