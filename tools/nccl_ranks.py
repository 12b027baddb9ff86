"""Run libgts's real multi-rank path (NCCL communicator, one process per rank):
rank r on GPU r % device_count.  With one GPU both ranks share it, which NCCL
2.28 refuses (ncclCommInitRank: invalid usage -- both ranks then fail the call
with GTS_ENCCL, no hang; profiles/r02_two_ranks_one_gpu.txt); with two or more
GPUs this is the real NCCL / CUDA IPC path end to end.

Each rank builds its own owner-filtered pages and runs BFS / PageRank / SSSP / WCC
under Strategy-P and Strategy-S (routed, and GTS_ROUTE_PEER over CUDA IPC), then
compares with the oracle.  Prints one JSON line per rank.

    python tools/nccl_two_ranks_one_gpu.py [--scale 14]
"""
import argparse
import json
import os
import socket
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def worker(rank, world, port, scale, q):
    import numpy as np
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import inputs
    import oracle
    import paper_conf_sigmod_0002apsk16_b200 as G
    res = {"rank": rank}
    try:
        obj = [G.gts_get_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        import torch
        ctx = G.gts_context_create(rank % max(1, torch.cuda.device_count()), rank, world, obj[0])
        g = inputs.rmat(scale)
        w = inputs.edge_weights(g)
        for sname, strat, peer in (("P", 0, False), ("S", 1, False), ("S_peer", 1, True), ("S_BCAST", 2, False)):
            own = (rank, world, strat)
            gr = G.gts_build_pages(g.row_ptr, g.col, page_bytes=4096, order=True, owner=own)
            grw = G.gts_build_pages(g.row_ptr, g.col, w, page_bytes=8192, owner=own)
            grs = G.gts_build_pages(g.row_ptr, g.col, page_bytes=4096, symmetric=True, owner=own)
            kw = dict(strategy=strat)
            lv, _ = G.gts_bfs(ctx, gr, 0, route_peer=peer, **kw)
            res[sname + "_bfs"] = bool(np.array_equal(lv, oracle.bfs(g.row_ptr, g.col, 0)))
            x, _ = G.gts_pagerank(ctx, gr, 10, 0.85, route_peer=peer, **kw)
            ref = oracle.pagerank(g.row_ptr, g.col, 10, 0.85)
            res[sname + "_pr_max_rel"] = float(np.max(np.abs(x - ref) / ref))
            d, _ = G.gts_sssp(ctx, grw, 0, route_peer=peer, **kw)
            res[sname + "_sssp"] = bool(np.array_equal(d, oracle.sssp(g.row_ptr, g.col, w, 0)))
            lab, _ = G.gts_wcc(ctx, grs if strat == 1 else gr, route_peer=peer, **kw)
            res[sname + "_wcc"] = bool(np.array_equal(lab, oracle.wcc(g.row_ptr, g.col)))
        ctx.free()
    except Exception as e:  # pragma: no cover
        res["error"] = repr(e)
    q.put(res)
    dist.destroy_process_group()


def main():
    import torch.multiprocessing as mp
    ap = argparse.ArgumentParser()
    ap.add_argument("--scale", type=int, default=14)
    ap.add_argument("--world", type=int, default=2)
    a = ap.parse_args()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    procs = [ctx.Process(target=worker, args=(r, a.world, port, a.scale, q)) for r in range(a.world)]
    for p in procs:
        p.start()
    for _ in procs:
        print(json.dumps(q.get(timeout=600)), flush=True)
    for p in procs:
        p.join(60)


if __name__ == "__main__":
    main()
