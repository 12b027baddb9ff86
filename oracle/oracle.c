/*
 * oracle/oracle.c -- TEST INFRASTRUCTURE ONLY.
 *
 * A plain, slow CPU implementation of what the GTS hot path computes, over
 * CSR (never over the slotted pages, except the page decoder at
 * the bottom, which reads page bytes by the format's definition).  It shares
 * no code, header, table or constant generator with the CUDA path
 * (paper_conf_sigmod_0002apsk16_b200/csrc) and neither side includes the
 * other.  Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load it.
 *
 * Citations: P:L = /root/reference/PAPER.md line L (SIGMOD'16 GTS paper).
 * Readings R# = DESIGN.md "Readings of the paper".
 *
 * Every function here is pinned by tests/test_oracle_*.py to something other
 * than itself (brute force, closed forms, scipy / networkx / numpy library
 * routines, invariants); see DESIGN.md "Oracle pins".
 *
 * Built twice: liboracle.so (plain, single-threaded: the
 * pragmas below are ignored) and liboracle_omp.so (-fopenmp).  The OpenMP
 * pragmas only split loops whose iterations write disjoint outputs, each
 * computed in the same fixed order as the plain build (PageRank: y[v] sums
 * its in-edges in ascending u), so the two builds are byte-identical
 * (tests/test_oracle_pagerank.py::test_openmp_build_byte_identical).
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#define UNREACHED 0xFFFFFFFFu

/* ------------------------------------------------------------------ BFS ---
 * Level-synchronous BFS over OUTGOING edges (ADJLIST = outgoing edges, P:538;
 * Alg 2 lines 9,17-18 and Alg 3 lines 5,9-10: a vertex at
 * curLevel sets every unvisited neighbour (LV = NULL) to curLevel+1).
 * Written as the textbook FIFO-queue BFS, whose levels equal the hop distance
 * from src.  NULL = UINT32_MAX (R7). */
int oracle_bfs(uint64_t n, const uint64_t* row_ptr, const uint32_t* col, uint64_t src,
               uint32_t* level /* n */) {
    if (src >= n) return -1;
    for (uint64_t v = 0; v < n; ++v) level[v] = UNREACHED;
    uint32_t* queue = (uint32_t*)malloc((n ? n : 1) * sizeof(uint32_t));
    if (!queue) return -2;
    uint64_t head = 0, tail = 0;
    level[src] = 0;
    queue[tail++] = (uint32_t)src;
    while (head < tail) {
        uint32_t u = queue[head++];
        for (uint64_t k = row_ptr[u]; k < row_ptr[u + 1]; ++k) {
            uint32_t v = col[k];
            if (level[v] == UNREACHED) {
                level[v] = level[u] + 1;
                queue[tail++] = v;
            }
        }
    }
    free(queue);
    return 0;
}

/* Level-synchronous BFS: the same hop levels as oracle_bfs, organised the way
 * Alg 1 drives the GPU (level by level, every vertex of the current
 * level L sets its unvisited out-neighbours to L+1, Alg 2 lines 17-18).  The
 * level sets are unique, so the result equals the FIFO-queue BFS (pinned in
 * tests/test_oracle_bfs.py).  Written so the OpenMP build splits each level's
 * frontier over the host cores (the all-core CPU baseline of SURVEY 8(d)): a
 * compare-and-swap on level[v] lets exactly one discoverer append v to the
 * next frontier. */
int oracle_bfs_levelsync(uint64_t n, const uint64_t* row_ptr, const uint32_t* col, uint64_t src,
                         uint32_t* level /* n */) {
    if (src >= n) return -1;
    for (uint64_t v = 0; v < n; ++v) level[v] = UNREACHED;
    uint32_t* cur = (uint32_t*)malloc((n ? n : 1) * sizeof(uint32_t));
    uint32_t* nxt = (uint32_t*)malloc((n ? n : 1) * sizeof(uint32_t));
    if (!cur || !nxt) return -2;
    level[src] = 0;
    cur[0] = (uint32_t)src;
    uint64_t ncur = 1;
    for (uint32_t L = 0; ncur > 0; ++L) {
        uint64_t nnext = 0;
        #pragma omp parallel
        {
            uint32_t buf[1024];
            uint64_t nb = 0;
            #pragma omp for schedule(dynamic, 64)
            for (uint64_t i = 0; i < ncur; ++i) {
                uint32_t u = cur[i];
                for (uint64_t k = row_ptr[u]; k < row_ptr[u + 1]; ++k) {
                    uint32_t v = col[k];
                    if (level[v] == UNREACHED && __sync_bool_compare_and_swap(&level[v], UNREACHED, L + 1)) {
                        buf[nb++] = v;
                        if (nb == 1024) {
                            uint64_t at = __atomic_fetch_add(&nnext, nb, __ATOMIC_RELAXED);
                            memcpy(nxt + at, buf, nb * sizeof(uint32_t));
                            nb = 0;
                        }
                    }
                }
            }
            if (nb) {
                uint64_t at = __atomic_fetch_add(&nnext, nb, __ATOMIC_RELAXED);
                memcpy(nxt + at, buf, nb * sizeof(uint32_t));
            }
        }
        uint32_t* t = cur; cur = nxt; nxt = t;
        ncur = nnext;
    }
    free(cur); free(nxt);
    return 0;
}

/* Threads the OpenMP build runs with (1 in the plain build). */
int oracle_num_threads(void) {
#ifdef _OPENMP
    int t = 1;
    #pragma omp parallel
    {
        #pragma omp single
        t = omp_get_num_threads();
    }
    return t;
#else
    return 1;
#endif
}

/* ------------------------------------------------------------- PageRank ---
 * PageRank as the GTS kernels compute it (Alg 4/5; P:1528-1532;
 * P:338), written as its plain definition in fp64:
 *   x^0_v = 1/n                                                   (R2)
 *   D^t   = sum of x^{t-1}_u over u with outdeg(u) = 0            (R3)
 *   x^t_v = (1-d)/n + d * ( sum_{edges u->v} x^{t-1}_u / outdeg(u)
 *                           + [dangling_uniform] D^t / n )
 * The edge sum runs over in-edges with multiplicity (R5), in ascending u
 * ("pull order") so the result is deterministic.  The in-edge lists are built
 * here by a counting sort (own transpose).  dangling_uniform = 0 reproduces the
 * paper literally (the mass of dangling vertices leaks, R3). */
int oracle_pagerank(uint64_t n, const uint64_t* row_ptr, const uint32_t* col, uint32_t iters,
                    double d, int dangling_uniform, double* x_out /* n */) {
    if (n == 0) return 0;
    uint64_t m = row_ptr[n];
    uint64_t* in_ptr = (uint64_t*)calloc(n + 1, sizeof(uint64_t));
    uint32_t* in_src = (uint32_t*)malloc((m ? m : 1) * sizeof(uint32_t));
    double* x = x_out;
    double* y = (double*)malloc(n * sizeof(double));
    double* contrib = (double*)malloc(n * sizeof(double));
    if (!in_ptr || !in_src || !y || !contrib) return -2;
    for (uint64_t k = 0; k < m; ++k) in_ptr[col[k] + 1]++;
    for (uint64_t v = 0; v < n; ++v) in_ptr[v + 1] += in_ptr[v];
    uint64_t* cur = (uint64_t*)malloc(n * sizeof(uint64_t));
    memcpy(cur, in_ptr, n * sizeof(uint64_t));
    for (uint64_t u = 0; u < n; ++u)               /* ascending u => each in-list ascending */
        for (uint64_t k = row_ptr[u]; k < row_ptr[u + 1]; ++k) in_src[cur[col[k]]++] = (uint32_t)u;
    free(cur);

    for (uint64_t v = 0; v < n; ++v) x[v] = 1.0 / (double)n;
    for (uint32_t t = 0; t < iters; ++t) {
        double D = 0.0;                            /* sequential: fixed summation order */
        for (uint64_t u = 0; u < n; ++u)
            if (row_ptr[u + 1] == row_ptr[u]) D += x[u];
        #pragma omp parallel for schedule(static)
        for (uint64_t u = 0; u < n; ++u) {
            uint64_t deg = row_ptr[u + 1] - row_ptr[u];
            contrib[u] = deg == 0 ? 0.0 : x[u] / (double)deg;
        }
        double base = (1.0 - d) / (double)n + (dangling_uniform ? d * D / (double)n : 0.0);
        #pragma omp parallel for schedule(dynamic, 4096)
        for (uint64_t v = 0; v < n; ++v) {
            double s = 0.0;
            for (uint64_t k = in_ptr[v]; k < in_ptr[v + 1]; ++k) s += contrib[in_src[k]];
            y[v] = base + d * s;
        }
        #pragma omp parallel for schedule(static)
        for (uint64_t v = 0; v < n; ++v) x[v] = y[v];
    }
    free(in_ptr); free(in_src); free(y); free(contrib);
    return 0;
}

/* ----------------------------------------------------------------- SSSP ---
 * Single-source shortest paths over out-edges with u32 weights (R11): the
 * paper lists SSSP among the BFS-like algorithms run by GTS
 * but gives no kernel; the oracle is the textbook Dijkstra with a binary heap
 * and u64 distances.  dist = UINT32_MAX when unreached; returns -6
 * (overflow) if a reachable distance is >= 2^32-1. */
typedef struct { uint64_t key; uint32_t v; } heap_item;

static void heap_push(heap_item* h, uint64_t* sz, heap_item it) {
    uint64_t i = (*sz)++;
    h[i] = it;
    while (i > 0) {
        uint64_t p = (i - 1) / 2;
        if (h[p].key <= h[i].key) break;
        heap_item t = h[p]; h[p] = h[i]; h[i] = t; i = p;
    }
}

static heap_item heap_pop(heap_item* h, uint64_t* sz) {
    heap_item top = h[0];
    h[0] = h[--(*sz)];
    uint64_t i = 0;
    for (;;) {
        uint64_t l = 2 * i + 1, r = l + 1, s = i;
        if (l < *sz && h[l].key < h[s].key) s = l;
        if (r < *sz && h[r].key < h[s].key) s = r;
        if (s == i) break;
        heap_item t = h[s]; h[s] = h[i]; h[i] = t; i = s;
    }
    return top;
}

int oracle_sssp(uint64_t n, const uint64_t* row_ptr, const uint32_t* col, const uint32_t* w,
                uint64_t src, uint32_t* dist_out /* n */) {
    if (src >= n) return -1;
    uint64_t m = row_ptr[n];
    uint64_t* dist = (uint64_t*)malloc(n * sizeof(uint64_t));
    heap_item* h = (heap_item*)malloc((m + 1) * sizeof(heap_item));
    if (!dist || !h) return -2;
    const uint64_t INF = ~0ULL;
    for (uint64_t v = 0; v < n; ++v) dist[v] = INF;
    uint64_t sz = 0;
    dist[src] = 0;
    heap_item s0 = {0, (uint32_t)src};
    heap_push(h, &sz, s0);
    while (sz > 0) {
        heap_item it = heap_pop(h, &sz);
        if (it.key != dist[it.v]) continue;           /* stale entry */
        uint32_t u = it.v;
        for (uint64_t k = row_ptr[u]; k < row_ptr[u + 1]; ++k) {
            uint64_t nd = dist[u] + (uint64_t)w[k];
            if (nd < dist[col[k]]) {
                dist[col[k]] = nd;
                heap_item ni = {nd, col[k]};
                heap_push(h, &sz, ni);
            }
        }
    }
    int rc = 0;
    for (uint64_t v = 0; v < n; ++v) {
        if (dist[v] == INF) dist_out[v] = UNREACHED;
        else if (dist[v] >= (uint64_t)UNREACHED) { rc = -6; dist_out[v] = UNREACHED; }
        else dist_out[v] = (uint32_t)dist[v];
    }
    free(dist); free(h);
    return rc;
}

/* ------------------------------------------------------------------ WCC ---
 * "Connected components" read as weakly connected components
 * of the directed graph, labelled by the minimum VID of the component (R12).
 * Textbook union-find over every edge taken as undirected; the union always
 * makes the smaller root the parent, so each root is its component's min VID. */
static uint32_t uf_find(uint32_t* parent, uint32_t v) {
    while (parent[v] != v) {
        parent[v] = parent[parent[v]];                /* path halving */
        v = parent[v];
    }
    return v;
}

int oracle_wcc(uint64_t n, const uint64_t* row_ptr, const uint32_t* col, uint32_t* label /* n */) {
    for (uint64_t v = 0; v < n; ++v) label[v] = (uint32_t)v;
    for (uint64_t u = 0; u < n; ++u) {
        for (uint64_t k = row_ptr[u]; k < row_ptr[u + 1]; ++k) {
            uint32_t a = uf_find(label, (uint32_t)u), b = uf_find(label, col[k]);
            if (a < b) label[b] = a;
            else if (b < a) label[a] = b;
        }
    }
    for (uint64_t v = 0; v < n; ++v) label[v] = uf_find(label, (uint32_t)v);
    return 0;
}

/* ---------------------------------------------------------- page decoder ---
 * Reads slotted pages by the format's definition ("records grow forward
 * from the start of the page, slots grow backward from the end; a slot is
 * (VID, OFF); a record is (ADJLIST_SZ, ADJLIST)"; SP holds many
 * vertices, one high-degree vertex spans several LPs) with the concrete byte
 * layout fixed in include/gts.h ("Page layout"), and rebuilds CSR.
 *   footer (last 8 bytes):  u32 nslots, u32 kind (0 = SP, 1 = LP)
 *   LP adds before it:       u32 total_deg, u32 chunk_idx
 *   slot k (k = 0,1,..):     at page_end - footer - 8(k+1): u32 vid, u32 off
 *   record at off:           u32 sz, u32 adj[sz]            (unweighted)
 *                            u32 sz, u32 0, (u32 adj, u32 w)[sz]  (weighted)
 * Entry encoding 0 = VID32; 1 = PID16_SLOT16 (ADJ_PID << 16 | ADJ_OFF), decoded
 * as RVT[ADJ_PID].START_VID + ADJ_OFF (App A) where START_VID of a page
 * is the VID of its slot 0.
 * Output: row_ptr[n+1] with n = 1 + max VID seen; col/w arrays (capacity m_cap).
 * Returns m, or a negative error. */
static uint32_t rd32(const uint8_t* p) { uint32_t x; memcpy(&x, p, 4); return x; }

int64_t oracle_decode_pages(const uint8_t* pages, uint64_t num_pages, uint64_t page_bytes,
                            int entry_encoding, int weighted, uint64_t n,
                            uint64_t* row_ptr /* n+1 */, uint32_t* col, uint32_t* w, uint64_t m_cap) {
    uint32_t* start_vid = (uint32_t*)malloc((num_pages ? num_pages : 1) * sizeof(uint32_t));
    uint64_t* deg = (uint64_t*)calloc(n + 1, sizeof(uint64_t));
    if (!start_vid || !deg) return -2;
    /* pass 1: RVT (START_VID per page) and per-vertex degrees */
    for (uint64_t p = 0; p < num_pages; ++p) {
        const uint8_t* pg = pages + p * page_bytes;
        const uint8_t* end = pg + page_bytes;
        uint32_t kind = rd32(end - 4), nslots = rd32(end - 8);
        uint64_t footer = kind == 1 ? 16 : 8;
        if (nslots == 0) { free(start_vid); free(deg); return -3; }
        start_vid[p] = rd32(end - footer - 8);
        for (uint32_t k = 0; k < nslots; ++k) {
            const uint8_t* s = end - footer - 8 * (uint64_t)(k + 1);
            uint32_t vid = rd32(s), off = rd32(s + 4);
            if (vid >= n) { free(start_vid); free(deg); return -4; }
            deg[vid] += rd32(pg + off);
        }
    }
    row_ptr[0] = 0;
    for (uint64_t v = 0; v < n; ++v) row_ptr[v + 1] = row_ptr[v] + deg[v];
    if (row_ptr[n] > m_cap) { free(start_vid); free(deg); return -5; }
    for (uint64_t v = 0; v < n; ++v) deg[v] = row_ptr[v];      /* reuse as cursor */
    /* pass 2: adjacency, pages in ID order (LP chunks of a vertex are in order) */
    for (uint64_t p = 0; p < num_pages; ++p) {
        const uint8_t* pg = pages + p * page_bytes;
        const uint8_t* end = pg + page_bytes;
        uint32_t kind = rd32(end - 4), nslots = rd32(end - 8);
        uint64_t footer = kind == 1 ? 16 : 8;
        for (uint32_t k = 0; k < nslots; ++k) {
            const uint8_t* s = end - footer - 8 * (uint64_t)(k + 1);
            uint32_t vid = rd32(s), off = rd32(s + 4);
            uint32_t sz = rd32(pg + off);
            uint64_t first = weighted ? 8 : 4, stride = weighted ? 8 : 4;   /* entries after the header */
            for (uint32_t i = 0; i < sz; ++i) {
                uint32_t e = rd32(pg + off + first + stride * (uint64_t)i);
                uint32_t v;
                if (entry_encoding == 1) {
                    uint32_t pid = e >> 16, slot = e & 0xFFFFu;
                    if (pid >= num_pages) { free(start_vid); free(deg); return -4; }
                    v = start_vid[pid] + slot;
                } else {
                    v = e;
                }
                col[deg[vid]] = v;
                if (weighted && w) w[deg[vid]] = rd32(pg + off + first + stride * (uint64_t)i + 4);
                deg[vid]++;
            }
        }
    }
    int64_t m = (int64_t)row_ptr[n];
    free(start_vid); free(deg);
    return m;
}

/* ------------------------------------------------------------------- BC ---
 * Betweenness centrality restricted to a set of sources (the paper runs BC as
 * a BFS-like algorithm on GTS, Fig 13c; no kernel is given).  Textbook
 * Brandes (2001) for unweighted directed multigraphs over out-edges, fp64:
 *   for each source s: BFS levels d and path counts sigma (sigma[s] = 1,
 *   sigma[w] += sigma[v] over every edge v->w with d[w] = d[v] + 1, parallel
 *   edges counted with multiplicity); then in non-increasing d order
 *   delta[v] = sum over edges v->w with d[w] = d[v] + 1 of
 *              sigma[v] / sigma[w] * (1 + delta[w]);
 *   bc[v] += delta[v] for v != s.
 * bc_out[n] is accumulated over the k sources (not normalised). */
int oracle_bc(uint64_t n, const uint64_t* row_ptr, const uint32_t* col, const uint32_t* sources, uint64_t k,
              double* bc_out) {
    uint32_t* d = (uint32_t*)malloc(n * sizeof(uint32_t));
    double* sigma = (double*)malloc(n * sizeof(double));
    double* delta = (double*)malloc(n * sizeof(double));
    uint32_t* order = (uint32_t*)malloc((n ? n : 1) * sizeof(uint32_t));
    if (!d || !sigma || !delta || !order) return -2;
    for (uint64_t v = 0; v < n; ++v) bc_out[v] = 0.0;
    for (uint64_t si = 0; si < k; ++si) {
        uint32_t s = sources[si];
        if (s >= n) { free(d); free(sigma); free(delta); free(order); return -1; }
        for (uint64_t v = 0; v < n; ++v) { d[v] = UNREACHED; sigma[v] = 0.0; delta[v] = 0.0; }
        uint64_t head = 0, tail = 0;
        d[s] = 0; sigma[s] = 1.0; order[tail++] = s;
        while (head < tail) {                       /* BFS: order = vertices by non-decreasing d */
            uint32_t v = order[head++];
            for (uint64_t e = row_ptr[v]; e < row_ptr[v + 1]; ++e) {
                uint32_t w = col[e];
                if (d[w] == UNREACHED) { d[w] = d[v] + 1; order[tail++] = w; }
                if (d[w] == d[v] + 1) sigma[w] += sigma[v];
            }
        }
        for (uint64_t i = tail; i-- > 0;) {         /* dependencies in non-increasing d */
            uint32_t v = order[i];
            for (uint64_t e = row_ptr[v]; e < row_ptr[v + 1]; ++e) {
                uint32_t w = col[e];
                if (d[w] == d[v] + 1) delta[v] += sigma[v] / sigma[w] * (1.0 + delta[w]);
            }
            if (v != s) bc_out[v] += delta[v];
        }
    }
    free(d); free(sigma); free(delta); free(order);
    return 0;
}
