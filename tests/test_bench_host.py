"""bench.py host logic on CPU: the N > 1 graph sharing through /dev/shm (gloo,
world_size 2) and the reference arm's JSON line."""
import json
import os
import socket
import subprocess
import sys

import numpy as np
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, port, out):
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=2)
    import bench
    import inputs

    class A:
        workload = "rmat"
        scale = 10

    g = bench.make_graph(A, rank, 2, dist)
    ref = inputs.rmat(10)
    ok = bool(np.array_equal(g.col, ref.col) and np.array_equal(g.row_ptr, ref.row_ptr))
    bench.drop_shared_graph(A, rank, 2, dist)
    out[rank] = ok
    dist.destroy_process_group()


def test_graph_shared_across_ranks():
    ctx = mp.get_context("spawn")
    out = ctx.Manager().dict()
    port = _port()
    ps = [ctx.Process(target=_worker, args=(r, port, out)) for r in range(2)]
    for p in ps:
        p.start()
    for p in ps:
        p.join(120)
    assert all(p.exitcode == 0 for p in ps) and out[0] and out[1]
    assert not os.path.exists(f"/dev/shm/gts_bench_rmat_10_{port}_rp.npy")


def test_reference_arm_line():
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--scale", "14",
                        "--steps", "2", "--warmup", "1"], capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stderr
    line = json.loads(r.stdout.strip().splitlines()[-1])
    assert line["impl"] == "reference" and line["value"] > 0 and line["unit"] == "GTEPS"
    assert line["cpu_baseline"]["kind"] == "oracle" and line["e2e"]["h2d_bytes_per_step"] == 0


def test_bfs_algorithmic_bytes_hand_graph():
    """B_BFS of SURVEY 8(d) on a hand graph: 0->1, 0->2, 1->2, vertex 3 isolated, one SP
    page of 4 slots.  Levels 0 and 1 each activate that page (4 bits = 0.5 B each);
    3 reached vertices x 12 B (slot offset + ADJLIST_SZ + LV... see bench.py) and 3
    traversed edges x (4 B adjacency + 4 B visited test); 3 LV writes x 4 B."""
    sys.path.insert(0, ROOT)
    import bench
    import inputs
    import oracle
    import paper_conf_sigmod_0002apsk16_b200 as G
    g = inputs.from_edges(4, [(0, 1), (0, 2), (1, 2)])
    gr = G.gts_build_pages(g.row_ptr, g.col, page_bytes=256)
    lv = oracle.bfs(g.row_ptr, g.col, 0)
    b, parts = bench.bfs_algorithmic_bytes(lv, g.row_ptr, gr)
    assert parts["edges"] == 3 and parts["reached"] == 3 and parts["active_page_levels"] == 2
    assert b == 0.5 + 0.5 + 12 * 3 + 4 * 3 + 4 * 3 + 4 * 3
    # degree-ordered pages give the same bytes (the directory is in internal IDs)
    go = G.gts_build_pages(g.row_ptr, g.col, page_bytes=256, order=True)
    assert bench.bfs_algorithmic_bytes(lv, g.row_ptr, go)[0] == b
