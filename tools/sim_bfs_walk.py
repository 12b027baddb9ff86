"""CPU model of the BFS page walk on degree-ordered RMAT pages (no GPU).

For every BFS level it counts what the expansion kernel's dense-tile walk does
per 128-word warp window (expand.cuh dense_tile_ww): how many words are edges
of selected vertices that need the visited probe (dst >= the all-visited
prefix, "flagged"), how many windows have none, and the largest number of
flagged words one lane (4 consecutive words) holds -- the loop count of a
per-word owner search.  Page boundaries are ignored (tiles of 512 consecutive
vertices over one record stream).

    python tools/sim_bfs_walk.py --scale 24
"""
import argparse
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--scale", type=int, default=24)
    ap.add_argument("--tile", type=int, default=512)
    args = ap.parse_args()
    import inputs
    g = inputs.rmat(args.scale)
    n = g.n
    deg = np.diff(g.row_ptr).astype(np.int64)
    indeg = np.bincount(g.col, minlength=n)
    # descending in-degree, ties by VID (builder.cpp)
    order = np.lexsort((np.arange(n), -indeg))          # internal -> caller
    new_of_old = np.empty(n, np.int64)
    new_of_old[order] = np.arange(n)
    ideg = deg[order]
    irow = np.zeros(n + 1, np.int64)
    irow[1:] = np.cumsum(ideg)
    # columns in internal order, each row sorted
    starts = g.row_ptr[:-1].astype(np.int64)[order]
    idx = np.repeat(starts - irow[:-1], ideg) + np.arange(irow[-1])
    icol = new_of_old[g.col[idx]].astype(np.int64)
    rowid = np.repeat(np.arange(n), ideg)
    o = np.lexsort((icol, rowid))
    icol = icol[o]
    del o, idx
    # record stream: header word then deg entries
    woff = np.zeros(n + 1, np.int64)
    woff[1:] = np.cumsum(1 + ideg)
    src = new_of_old[0]
    lv = np.full(n, -1, np.int64)
    lv[src] = 0
    front = np.zeros(n, bool)
    front[src] = True
    visited = front.copy()
    T = args.tile
    ntile = (n + T - 1) // T
    L = 0
    print(f"RMAT-{args.scale}: n={n} m={len(icol)} src(internal)={src}")
    print("lvl frontier  vprefix  edges_sel  flagged%  dense_t sparse_t  dense_win  win_no_flag%  "
          "E[maxlane]  sparse_edges  sparse_flag%")
    while front.any():
        fv = np.nonzero(front)[0]
        # all-visited prefix in whole 32-bit words
        nz = np.nonzero(~visited)[0]
        vp = (nz[0] // 32) * 32 if len(nz) else n
        sel_e = ideg * front
        tile_sel = np.add.reduceat(sel_e, np.arange(0, n, T))
        tile_w = np.add.reduceat(1 + ideg, np.arange(0, n, T))
        tile_act = np.add.reduceat(front.astype(np.int64), np.arange(0, n, T)) > 0
        dense = tile_act & (8 * tile_sel >= 6 * tile_w)
        sparse = tile_act & ~dense
        # per-word flags over the dense tiles' record regions
        e_front = np.repeat(front, ideg)
        flag_e = e_front & (icol >= vp)
        nflag = flag_e.sum()
        dw = 0
        noflag = 0
        maxlane_sum = 0
        allsel_e = 0
        dense_e = 0
        for t in np.nonzero(dense)[0]:
            v0, v1 = t * T, min(n, (t + 1) * T)
            has = ideg[v0:v1] > 0
            dense_e += int(sel_e[v0:v1].sum())
            if np.all(visited[v0:v1][has]):        # every vertex with edges visited: no selection needed
                allsel_e += int(sel_e[v0:v1].sum())
            W0, W1 = woff[v0], woff[v1]
            words = np.zeros(W1 - W0, bool)
            e0, e1 = irow[v0], irow[v1]
            # word index of edge k of vertex v = woff[v] + 1 + (k - irow[v])
            ev = np.repeat(np.arange(v0, v1), ideg[v0:v1])
            wi = woff[ev] + 1 + (np.arange(e0, e1) - irow[ev]) - W0
            words[wi[flag_e[e0:e1]]] = True
            base = W0 & ~3
            pad0 = W0 - base
            nw = ((W1 - base + 127) // 128) * 128
            ww = np.zeros(nw, bool)
            ww[pad0:pad0 + len(words)] = words
            win = ww.reshape(-1, 32, 4).sum(axis=2)          # flagged words per lane
            dw += win.shape[0]
            noflag += int((win.max(axis=1) == 0).sum())
            maxlane_sum += int(win.max(axis=1).sum())
        sp_tiles = np.nonzero(sparse)[0]
        sp_mask = np.zeros(n, bool)
        for t in sp_tiles:
            sp_mask[t * T:(t + 1) * T] = True
        sp_e = np.repeat(front & sp_mask, ideg)
        spn = int(sp_e.sum())
        spf = int((sp_e & (icol >= vp)).sum())
        print(f"{L:3d} {len(fv):9d} {vp:9d} {int(sel_e.sum()):10d} {100 * nflag / max(1, sel_e.sum()):8.1f} "
              f"{int(dense.sum()):8d} {int(sparse.sum()):8d} {dw:10d} {100 * noflag / max(1, dw):12.1f} "
              f"{maxlane_sum / max(1, dw):11.2f} {spn:13d} {100 * spf / max(1, spn):12.1f}  "
              f"dense_e {dense_e} all_visited_e {allsel_e} ({100 * allsel_e / max(1, dense_e):.1f}%) "
              f"maxdeg {int(ideg.max())}")
        # next level
        nb = icol[np.repeat(front, ideg)]
        nxt = np.zeros(n, bool)
        nxt[nb] = True
        nxt &= ~visited
        visited |= nxt
        front = nxt
        L += 1


if __name__ == "__main__":
    main()
