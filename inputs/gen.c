/*
 * inputs/gen.c -- seeded synthetic graph generators (the ONE module shared by
 * the oracle side and the CUDA side of the tests/bench).
 *
 * This file holds no arithmetic of the GTS method (no BFS, PageRank, SSSP,
 * WCC, no page format).  It only draws graphs, as CSR:
 *     row_ptr : uint64_t[n+1]   (row_ptr[0] = 0, row_ptr[n] = m)
 *     col_idx : uint32_t[m]     destination VIDs; each row sorted ascending
 *     weights : uint32_t[m]     optional, 1..255 (SSSP)
 * Duplicates (multi-edges) and self-loops are kept (reading R5).
 *
 * All random draws are counter based (splitmix64 of (seed, edge, level)), so the
 * graph is a pure function of the parameters, independent of thread count.
 *
 * RMAT  : Chakrabarti et al. [4] as used by GTS ("RMAT27..32,
 *         #edges = 16 x #vertices"); (a,b,c,d) = (0.57,0.19,0.19,0.05)
 *         (BASELINE.json north_star; reading R13).  No noise, no VID
 *         permutation, so low VIDs are hubs (this is what produces LPs).
 * Twitter-shaped : power-law out-degree sequence d_i = floor(C (i+i0)^-beta)
 *         (SURVEY.md section 8(d) C2), destinations drawn from an alias table
 *         of the same power law over a seeded VID permutation.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>
#include <omp.h>

static inline uint64_t splitmix64(uint64_t x) {
    x += 0x9E3779B97F4A7C15ULL;
    x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ULL;
    x = (x ^ (x >> 27)) * 0x94D049BB133111EBULL;
    return x ^ (x >> 31);
}

int gen_num_threads(void) { return omp_get_max_threads(); }

/* ---------------------------------------------------------------- RMAT --- */

typedef struct { uint64_t ta, tab, tabc; uint64_t seed_mix; int scale; } rmat_p;

/* Draw edge e: for each level (MSB first) pick a quadrant of the adjacency
 * matrix with probabilities a (0,0), b (0,1), c (1,0), d (1,1); row = src. */
static inline void rmat_edge(const rmat_p* p, uint64_t e, uint32_t* su, uint32_t* sv) {
    uint64_t u = 0, v = 0;
    uint64_t h = 0;
    for (int l = 0; l < p->scale; ++l) {
        uint64_t r;
        if ((l & 1) == 0) { h = splitmix64(p->seed_mix + ((e << 5) | (uint64_t)(l >> 1))); r = h >> 32; }
        else r = h & 0xFFFFFFFFULL;
        /* quadrant: [0,a) -> (0,0), [a,a+b) -> (0,1), [a+b,a+b+c) -> (1,0), else (1,1); branch-free */
        uint64_t ga = r >= p->ta, gab = r >= p->tab, gabc = r >= p->tabc;
        u = (u << 1) | gab;
        v = (v << 1) | (ga ^ gab ^ gabc);
    }
    *su = (uint32_t)u; *sv = (uint32_t)v;
}

static int cmp_u32(const void* a, const void* b) {
    uint32_t x = *(const uint32_t*)a, y = *(const uint32_t*)b;
    return (x > y) - (x < y);
}

static void sort_rows(uint64_t n, const uint64_t* row_ptr, uint32_t* col) {
    #pragma omp parallel for schedule(dynamic, 4096)
    for (int64_t i = 0; i < (int64_t)n; ++i) {
        uint64_t b = row_ptr[i], e = row_ptr[i + 1];
        uint64_t len = e - b;
        if (len < 2) continue;
        uint32_t* a = col + b;
        if (len <= 32) {
            for (uint64_t x = 1; x < len; ++x) {
                uint32_t k = a[x]; uint64_t y = x;
                while (y > 0 && a[y - 1] > k) { a[y] = a[y - 1]; --y; }
                a[y] = k;
            }
        } else {
            qsort(a, len, sizeof(uint32_t), cmp_u32);
        }
    }
}

/* exclusive scan of counts (u64[n]) into row_ptr (u64[n+1]) */
static void scan_counts(uint64_t n, const uint64_t* cnt, uint64_t* row_ptr) {
    int T = omp_get_max_threads();
    uint64_t* part = (uint64_t*)calloc((size_t)T + 1, sizeof(uint64_t));
    #pragma omp parallel num_threads(T)
    {
        int t = omp_get_thread_num(), nt = omp_get_num_threads();
        uint64_t lo = n * (uint64_t)t / nt, hi = n * (uint64_t)(t + 1) / nt, s = 0;
        for (uint64_t i = lo; i < hi; ++i) s += cnt[i];
        part[t + 1] = s;
        #pragma omp barrier
        #pragma omp single
        { for (int k = 1; k <= nt; ++k) part[k] += part[k - 1]; }
        s = part[t];
        for (uint64_t i = lo; i < hi; ++i) { row_ptr[i] = s; s += cnt[i]; }
        if (t == nt - 1) row_ptr[n] = s;
    }
    free(part);
}

/* Size query: n = 2^scale, m = edge_factor * n. */
int gen_rmat(int scale, uint64_t edge_factor, double a, double b, double c, uint64_t seed,
             uint64_t* row_ptr /* n+1 */, uint32_t* col /* m */) {
    if (scale < 1 || scale > 32) return -1;
    uint64_t n = 1ULL << scale, m = edge_factor * n;
    rmat_p p;
    const double two32 = 4294967296.0;
    p.ta = (uint64_t)(a * two32);
    p.tab = (uint64_t)((a + b) * two32);
    p.tabc = (uint64_t)((a + b + c) * two32);
    p.seed_mix = splitmix64(seed ^ 0x524D4154ULL /* "RMAT" */);
    p.scale = scale;
    uint64_t* cnt = (uint64_t*)calloc(n, sizeof(uint64_t));
    uint32_t* tmp = (uint32_t*)malloc(2 * m * sizeof(uint32_t));   /* one generation pass: (u, v) pairs */
    if (!cnt || !tmp) { free(cnt); free(tmp); return -2; }
    #pragma omp parallel for schedule(static, 65536)
    for (int64_t e = 0; e < (int64_t)m; ++e) {
        uint32_t u, v; rmat_edge(&p, (uint64_t)e, &u, &v);
        tmp[2 * e] = u; tmp[2 * e + 1] = v;
        __atomic_fetch_add(&cnt[u], 1, __ATOMIC_RELAXED);
    }
    scan_counts(n, cnt, row_ptr);
    memcpy(cnt, row_ptr, n * sizeof(uint64_t)); /* cursors */
    #pragma omp parallel for schedule(static, 65536)
    for (int64_t e = 0; e < (int64_t)m; ++e) {
        uint64_t pos = __atomic_fetch_add(&cnt[tmp[2 * e]], 1, __ATOMIC_RELAXED);
        col[pos] = tmp[2 * e + 1];
    }
    free(tmp);
    free(cnt);
    sort_rows(n, row_ptr, col);
    return 0;
}

/* Same graph as gen_rmat, without the (u, v) pair buffer: the edges are drawn
 * twice (count pass, fill pass).  For scales whose pair buffer (8 m bytes)
 * does not fit in host memory next to the CSR. */
int gen_rmat_lean(int scale, uint64_t edge_factor, double a, double b, double c, uint64_t seed,
                  uint64_t* row_ptr /* n+1 */, uint32_t* col /* m */) {
    if (scale < 1 || scale > 32) return -1;
    uint64_t n = 1ULL << scale, m = edge_factor * n;
    rmat_p p;
    const double two32 = 4294967296.0;
    p.ta = (uint64_t)(a * two32);
    p.tab = (uint64_t)((a + b) * two32);
    p.tabc = (uint64_t)((a + b + c) * two32);
    p.seed_mix = splitmix64(seed ^ 0x524D4154ULL /* "RMAT" */);
    p.scale = scale;
    uint64_t* cnt = (uint64_t*)calloc(n, sizeof(uint64_t));
    if (!cnt) return -2;
    #pragma omp parallel for schedule(static, 65536)
    for (int64_t e = 0; e < (int64_t)m; ++e) {
        uint32_t u, v; rmat_edge(&p, (uint64_t)e, &u, &v);
        __atomic_fetch_add(&cnt[u], 1, __ATOMIC_RELAXED);
    }
    scan_counts(n, cnt, row_ptr);
    memcpy(cnt, row_ptr, n * sizeof(uint64_t));
    #pragma omp parallel for schedule(static, 65536)
    for (int64_t e = 0; e < (int64_t)m; ++e) {
        uint32_t u, v; rmat_edge(&p, (uint64_t)e, &u, &v);
        uint64_t pos = __atomic_fetch_add(&cnt[u], 1, __ATOMIC_RELAXED);
        col[pos] = v;
    }
    free(cnt);
    sort_rows(n, row_ptr, col);
    return 0;
}

/* ------------------------------------------------------- Twitter-shaped --- */

/* degree sequence d_i = floor(C (i+i0)^-beta), C chosen so sum d = m; the
 * rounding deficit goes +1 to the first vertices (the top of the sequence). */
int gen_powerlaw_degrees(uint64_t n, uint64_t m, double beta, double i0, uint64_t* deg /* n */) {
    double lo = 0.0, hi = (double)m * 4.0 + 1.0;
    for (int it = 0; it < 200; ++it) {
        double C = 0.5 * (lo + hi);
        uint64_t s = 0;
        #pragma omp parallel for reduction(+:s)
        for (int64_t i = 0; i < (int64_t)n; ++i) s += (uint64_t)floor(C * pow((double)i + i0, -beta));
        if (s > m) hi = C; else lo = C;
    }
    uint64_t s = 0;
    #pragma omp parallel for reduction(+:s)
    for (int64_t i = 0; i < (int64_t)n; ++i) {
        deg[i] = (uint64_t)floor(lo * pow((double)i + i0, -beta));
        s += deg[i];
    }
    if (s > m) return -1;
    uint64_t deficit = m - s;
    for (uint64_t i = 0; deficit > 0; i = (i + 1) % n) { deg[i]++; deficit--; }
    return 0;
}

/* Vose alias table over weights w_i = (i+i0)^-beta */
static void build_alias(uint64_t n, double beta, double i0, float* prob, uint32_t* alias) {
    double* w = (double*)malloc(n * sizeof(double));
    double sum = 0;
    for (uint64_t i = 0; i < n; ++i) { w[i] = pow((double)i + i0, -beta); sum += w[i]; }
    uint32_t* small = (uint32_t*)malloc(n * sizeof(uint32_t));
    uint32_t* large = (uint32_t*)malloc(n * sizeof(uint32_t));
    uint64_t ns = 0, nl = 0;
    for (uint64_t i = 0; i < n; ++i) {
        w[i] = w[i] * (double)n / sum;
        if (w[i] < 1.0) small[ns++] = (uint32_t)i; else large[nl++] = (uint32_t)i;
    }
    while (ns > 0 && nl > 0) {
        uint32_t s = small[--ns], l = large[--nl];
        prob[s] = (float)w[s]; alias[s] = l;
        w[l] = (w[l] + w[s]) - 1.0;
        if (w[l] < 1.0) small[ns++] = l; else large[nl++] = l;
    }
    while (nl > 0) { uint32_t l = large[--nl]; prob[l] = 1.0f; alias[l] = l; }
    while (ns > 0) { uint32_t s = small[--ns]; prob[s] = 1.0f; alias[s] = s; }
    free(w); free(small); free(large);
}

int gen_twitter_like(uint64_t n, uint64_t m, double beta, double i0, uint64_t seed,
                     uint64_t* row_ptr /* n+1 */, uint32_t* col /* m */) {
    if (n == 0 || n > (1ULL << 32)) return -1;
    uint64_t* deg = (uint64_t*)malloc(n * sizeof(uint64_t));
    if (!deg) return -2;
    if (gen_powerlaw_degrees(n, m, beta, i0, deg) != 0) { free(deg); return -1; }
    scan_counts(n, deg, row_ptr);
    free(deg);
    float* prob = (float*)malloc(n * sizeof(float));
    uint32_t* alias = (uint32_t*)malloc(n * sizeof(uint32_t));
    uint32_t* perm = (uint32_t*)malloc(n * sizeof(uint32_t));
    if (!prob || !alias || !perm) return -2;
    build_alias(n, beta, i0, prob, alias);
    /* seeded Fisher-Yates permutation: in-weight rank r -> VID perm[r] */
    for (uint64_t i = 0; i < n; ++i) perm[i] = (uint32_t)i;
    uint64_t sm = splitmix64(seed ^ 0x5045524DULL);
    for (uint64_t i = n - 1; i > 0; --i) {
        uint64_t j = splitmix64(sm + i) % (i + 1);
        uint32_t t = perm[i]; perm[i] = perm[j]; perm[j] = t;
    }
    uint64_t dm = splitmix64(seed ^ 0x44535453ULL);
    #pragma omp parallel for schedule(static, 65536)
    for (int64_t e = 0; e < (int64_t)m; ++e) {
        uint64_t h = splitmix64(dm + (uint64_t)e);
        uint64_t k = (h >> 32) % n;
        float f = (float)(h & 0xFFFFFF) / 16777216.0f;
        uint32_t r = (f < prob[k]) ? (uint32_t)k : alias[k];
        col[e] = perm[r];
    }
    free(prob); free(alias); free(perm);
    sort_rows(n, row_ptr, col);
    return 0;
}

/* ------------------------------------------------------------- weights --- */

/* w(u,v) = 1 + (splitmix64(seed ^ (u<<32 ^ v)) mod 255): parallel edges share
 * a weight (reading R11). */
void gen_edge_weights(uint64_t n, const uint64_t* row_ptr, const uint32_t* col, uint64_t seed,
                      uint32_t* w /* m */) {
    #pragma omp parallel for schedule(dynamic, 4096)
    for (int64_t u = 0; u < (int64_t)n; ++u) {
        for (uint64_t k = row_ptr[u]; k < row_ptr[u + 1]; ++k) {
            uint64_t key = seed ^ (((uint64_t)u << 32) ^ (uint64_t)col[k]);
            w[k] = 1u + (uint32_t)(splitmix64(key) % 255u);
        }
    }
}

/* ------------------------------------------------------------ relabel --- */

/* Apply a vertex permutation to a CSR graph: vertex v becomes new_of_old[v];
 * out rows sorted.  (Input preparation for ordering experiments.) */
int gen_permute_csr(uint64_t n, const uint64_t* row_ptr, const uint32_t* col, const uint32_t* new_of_old,
                    uint64_t* out_row_ptr, uint32_t* out_col) {
    uint64_t* deg = (uint64_t*)malloc(n * sizeof(uint64_t));
    uint32_t* old_of_new = (uint32_t*)malloc(n * sizeof(uint32_t));
    if (!deg || !old_of_new) return -2;
    #pragma omp parallel for
    for (int64_t v = 0; v < (int64_t)n; ++v) {
        old_of_new[new_of_old[v]] = (uint32_t)v;
    }
    #pragma omp parallel for
    for (int64_t u = 0; u < (int64_t)n; ++u) deg[u] = row_ptr[old_of_new[u] + 1] - row_ptr[old_of_new[u]];
    scan_counts(n, deg, out_row_ptr);
    #pragma omp parallel for schedule(dynamic, 4096)
    for (int64_t u = 0; u < (int64_t)n; ++u) {
        uint64_t o = row_ptr[old_of_new[u]], b = out_row_ptr[u], e = out_row_ptr[u + 1];
        for (uint64_t k = 0; k < e - b; ++k) out_col[b + k] = new_of_old[col[o + k]];
    }
    free(deg); free(old_of_new);
    sort_rows(n, out_row_ptr, out_col);
    return 0;
}

/* new_of_old = rank of v by in-degree (descending, ties by VID) */
int gen_indegree_order(uint64_t n, const uint64_t* row_ptr, const uint32_t* col, uint32_t* new_of_old) {
    uint64_t m = row_ptr[n];
    uint32_t* indeg = (uint32_t*)calloc(n, sizeof(uint32_t));
    if (!indeg) return -2;
    #pragma omp parallel for schedule(static, 65536)
    for (int64_t k = 0; k < (int64_t)m; ++k) __atomic_fetch_add(&indeg[col[k]], 1u, __ATOMIC_RELAXED);
    /* counting sort by in-degree descending (stable in VID) */
    uint32_t maxd = 0;
    for (uint64_t v = 0; v < n; ++v) if (indeg[v] > maxd) maxd = indeg[v];
    uint64_t* bucket = (uint64_t*)calloc((size_t)maxd + 2, sizeof(uint64_t));
    for (uint64_t v = 0; v < n; ++v) bucket[maxd - indeg[v] + 1]++;
    for (uint64_t d = 1; d <= (uint64_t)maxd + 1; ++d) bucket[d] += bucket[d - 1];
    for (uint64_t v = 0; v < n; ++v) new_of_old[v] = (uint32_t)(bucket[maxd - indeg[v]]++);
    free(bucket); free(indeg);
    return 0;
}
