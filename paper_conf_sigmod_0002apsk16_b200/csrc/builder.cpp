// gts_build_pages: CSR -> slotted pages (SP/LP) + RVT.
//
// Paper: slotted page format P:64 (records forward from the start, slots
// backward from the end, slot = (VID, OFF), record = (ADJLIST_SZ, ADJLIST),
// VIDs consecutive within a page), SP/LP split P:66 + Fig 1,
// (p,q) physical IDs P:528-532, RVT P:1456-1486.  Byte layout: include/gts.h.
// Packing rule (R15): vertices in VID order, greedy; a vertex whose record +
// slot does not fit an empty SP becomes ceil(deg / cap_LP) LPs.
//
// Pure host code (no CUDA calls), OpenMP-parallel over pages.
#include <omp.h>

#include <algorithm>
#include <atomic>
#include <cstdlib>
#include <cstring>

#include "gts_internal.h"

namespace gts {

static std::atomic<uint64_t> g_next_uid{1};

void partition(const Graph* g, uint32_t strategy, int world, std::vector<int32_t>& owner,
               std::vector<uint64_t>& vrange) {
    const uint64_t P = g->num_pages;
    owner.assign(P, 0);
    vrange.assign(world + 1, g->n);
    vrange[0] = 0;
    if (world <= 1) return;
    if (strategy == GTS_STRATEGY_P) {
        for (uint64_t j = 0; j < P; ++j) owner[j] = (int32_t)(j % (uint64_t)world);   // h(j) = j mod N
        return;
    }
    // Strategy-S and S_BCAST share the WA ranges; under S_BCAST owner[j] is the
    // WA owner of the page's sources, but every rank processes every page.
    // Strategy-S: contiguous VID ranges cut at page boundaries (never inside an
    // LP run) with ~equal page counts; rank r owns WA[vrange[r], vrange[r+1]).
    uint64_t p = 0;
    for (int r = 0; r < world; ++r) {
        uint64_t target = (P * (uint64_t)(r + 1)) / (uint64_t)world;
        if (r == world - 1) target = P;
        uint64_t first = p;
        while (p < target || (p < P && p > 0 && g->kind[p] == GTS_PAGE_LP && g->lp_first[p] != (int64_t)p)) {
            owner[p] = r;
            ++p;
        }
        vrange[r] = first < P ? g->start_vid[first] : g->n;
        if (r == 0) vrange[0] = 0;
    }
    // ranks left without pages own an empty range at the end
    for (int r = 1; r <= world; ++r) vrange[r] = std::max(vrange[r], vrange[r - 1]);
    vrange[world] = g->n;
}


static inline void wr32(uint8_t* p, uint32_t v) { std::memcpy(p, &v, 4); }

static bool valid_page_bytes(uint32_t pb) {
    return pb >= 256 && (pb & (pb - 1)) == 0 && pb <= (1u << 30);
}

int plan_pages(uint64_t n, const uint64_t* row_ptr, bool weighted, uint32_t page_bytes,
               uint32_t entry_encoding, std::vector<PagePlanEntry>& plan, gts_graph_stats* st) {
    // record bytes: 4 + 4 deg (unweighted) or 8 + 8 deg (weighted: header sz, 0; (adj, w) pairs)
    const uint64_t words_per_edge = rec_edge_words(weighted), hdr_bytes = 4 * rec_hdr_words(weighted);
    const uint64_t sp_cap_bytes = page_bytes - kSpFooter;                    // records + slots
    const uint64_t lp_cap = (page_bytes - kLpFooter - kSlotBytes - hdr_bytes) / (4 * words_per_edge);
    const uint64_t max_slots = entry_encoding == GTS_ENTRY_PID16_SLOT16 ? 65536 : UINT32_MAX;
    if (lp_cap == 0) return fail(GTS_EINVAL, "page_bytes %u too small for one LP entry", page_bytes);
    plan.clear();
    uint64_t used_total = 0, n_sp = 0, n_lp = 0, n_lpv = 0, maxdeg = 0;
    PagePlanEntry cur{0, 0, GTS_PAGE_SP, -1, -1};
    uint64_t cur_used = 0;
    auto close_sp = [&]() {
        if (cur.nslots > 0) {
            plan.push_back(cur);
            used_total += cur_used + kSpFooter;
            ++n_sp;
        }
        cur.nslots = 0;
        cur_used = 0;
    };
    for (uint64_t v = 0; v < n; ++v) {
        uint64_t deg = row_ptr[v + 1] - row_ptr[v];
        if (deg > maxdeg) maxdeg = deg;
        if (deg >= (1ull << 32)) return fail(GTS_EOVERFLOW, "vertex %llu has degree >= 2^32", (unsigned long long)v);
        uint64_t need = hdr_bytes + 4 * words_per_edge * deg + kSlotBytes;
        if (need > sp_cap_bytes) {                                            // LP vertex
            close_sp();
            uint64_t chunks = (deg + lp_cap - 1) / lp_cap;
            int64_t first = (int64_t)plan.size();
            for (uint64_t c = 0; c < chunks; ++c) {
                uint64_t len = std::min(lp_cap, deg - c * lp_cap);
                plan.push_back(PagePlanEntry{(uint32_t)v, 1, GTS_PAGE_LP, first, first + (int64_t)chunks - 1});
                used_total += hdr_bytes + 4 * words_per_edge * len + kSlotBytes + kLpFooter;
            }
            n_lp += chunks;
            ++n_lpv;
            continue;
        }
        if (cur_used + need > sp_cap_bytes || cur.nslots >= max_slots) close_sp();
        if (cur.nslots == 0) cur.start_vid = (uint32_t)v;
        cur.nslots++;
        cur_used += need;
    }
    close_sp();
    if (entry_encoding == GTS_ENTRY_PID16_SLOT16 && plan.size() > 65536)
        return fail(GTS_EOVERFLOW, "PID16_SLOT16 encoding allows at most 65536 pages (%zu needed)", plan.size());
    if (st) {
        std::memset(st, 0, sizeof(*st));
        st->n = n;
        st->m = n ? row_ptr[n] : 0;
        st->num_pages = plan.size();
        st->n_sp = n_sp;
        st->n_lp = n_lp;
        st->n_lp_vertices = n_lpv;
        st->page_bytes = page_bytes;
        st->topo_bytes = (uint64_t)plan.size() * page_bytes;
        st->used_bytes = used_total;
        st->max_outdeg = maxdeg;
        st->weighted = weighted ? 1 : 0;
        st->entry_encoding = entry_encoding;
    }
    return GTS_OK;
}

// Hot-destination table: the kHotMax vertices of largest in-degree (>= kHotMinIndeg),
// hottest first, in a bucketed two-choice table (gts_internal.h).
static void build_hot_table(Graph& g, const uint32_t* col) {
    g.hot_keys.assign(kHotSlots, kHotEmpty);
    g.n_hot = 0;
    if (g.n == 0 || g.m == 0) return;
    std::vector<uint32_t> indeg(g.n, 0);
    #pragma omp parallel for schedule(static, 1 << 16)
    for (int64_t k = 0; k < (int64_t)g.m; ++k) __atomic_fetch_add(&indeg[col[k]], 1u, __ATOMIC_RELAXED);
    std::vector<std::vector<uint32_t>> cand_t(omp_get_max_threads());
    #pragma omp parallel
    {
        auto& c = cand_t[omp_get_thread_num()];
        #pragma omp for schedule(static)
        for (int64_t v = 0; v < (int64_t)g.n; ++v)
            if (indeg[v] >= kHotMinIndeg) c.push_back((uint32_t)v);
    }
    std::vector<uint32_t> cand;
    for (auto& c : cand_t) cand.insert(cand.end(), c.begin(), c.end());
    auto hotter = [&](uint32_t a, uint32_t b) { return indeg[a] != indeg[b] ? indeg[a] > indeg[b] : a < b; };
    size_t take = std::min<size_t>(cand.size(), kHotMax);
    std::partial_sort(cand.begin(), cand.begin() + take, cand.end(), hotter);
    for (size_t i = 0; i < take; ++i) {
        uint32_t v = cand[i];
        uint32_t bs[2] = {hot_h1(v), hot_h2(v)};
        for (uint32_t b : bs) {
            uint32_t* bucket = &g.hot_keys[b * kHotWays];
            int w = -1;
            for (uint32_t j = 0; j < kHotWays; ++j)
                if (bucket[j] == kHotEmpty) { w = (int)j; break; }
            if (w >= 0) { bucket[w] = v; g.n_hot++; break; }
        }
    }
}

}  // namespace gts

using namespace gts;

extern "C" int gts_plan_pages(uint64_t n, const uint64_t* row_ptr, int weighted, const gts_page_config* cfg,
                              gts_graph_stats* out) {
    clear_error();
    if (!row_ptr || !out) return fail(GTS_EINVAL, "NULL argument");
    if (n == 0) return fail(GTS_EINVAL, "n must be >= 1");
    if (n >= (1ull << 32)) return fail(GTS_EOVERFLOW, "n >= 2^32 (VID 0xFFFFFFFF is the NULL/empty sentinel)");
    uint32_t pb = (cfg && cfg->page_bytes) ? cfg->page_bytes : kDefaultPageBytes;
    uint32_t enc = cfg ? cfg->entry_encoding : GTS_ENTRY_VID32;
    if (!valid_page_bytes(pb)) return fail(GTS_EINVAL, "page_bytes %u must be a power of two in [256, 2^30]", pb);
    if (enc > GTS_ENTRY_PID16_SLOT16) return fail(GTS_EINVAL, "unknown entry encoding %u", enc);
    for (uint64_t v = 0; v < n; ++v)
        if (row_ptr[v + 1] < row_ptr[v]) return fail(GTS_EINVAL, "row_ptr not monotone at %llu", (unsigned long long)v);
    std::vector<PagePlanEntry> plan;
    return plan_pages(n, row_ptr, weighted != 0, pb, enc, plan, out);
}

// Symmetrised multigraph (GTS_BUILD_SYMMETRIC): row u = out(u) followed by in(u)
// (every edge u->v also stored as v->u), each row sorted (by (dst, weight)).
static void symmetrise(uint64_t n, const uint64_t* row_ptr, const uint32_t* col, const uint32_t* w,
                       std::vector<uint64_t>& s_row, std::vector<uint32_t>& s_col, std::vector<uint32_t>& s_w) {
    const uint64_t m = row_ptr[n];
    std::vector<uint64_t> indeg(n + 1, 0);
    for (uint64_t k = 0; k < m; ++k) indeg[col[k]]++;
    s_row.assign(n + 1, 0);
    for (uint64_t v = 0; v < n; ++v) s_row[v + 1] = s_row[v] + (row_ptr[v + 1] - row_ptr[v]) + indeg[v];
    s_col.resize(2 * m);
    if (w) s_w.resize(2 * m);
    std::vector<uint64_t> cur(n);
    for (uint64_t v = 0; v < n; ++v) {
        const uint64_t d = row_ptr[v + 1] - row_ptr[v];
        std::memcpy(s_col.data() + s_row[v], col + row_ptr[v], d * 4);
        if (w) std::memcpy(s_w.data() + s_row[v], w + row_ptr[v], d * 4);
        cur[v] = s_row[v] + d;
    }
    for (uint64_t u = 0; u < n; ++u)
        for (uint64_t k = row_ptr[u]; k < row_ptr[u + 1]; ++k) {
            const uint64_t at = cur[col[k]]++;
            s_col[at] = (uint32_t)u;
            if (w) s_w[at] = w[k];
        }
    #pragma omp parallel for schedule(dynamic, 1024)
    for (int64_t v = 0; v < (int64_t)n; ++v) {
        const uint64_t b = s_row[v], len = s_row[v + 1] - b;
        if (!w) {
            std::sort(s_col.begin() + b, s_col.begin() + b + len);
        } else {
            std::vector<std::pair<uint32_t, uint32_t>> e(len);
            for (uint64_t k = 0; k < len; ++k) e[k] = {s_col[b + k], s_w[b + k]};
            std::sort(e.begin(), e.end());
            for (uint64_t k = 0; k < len; ++k) {
                s_col[b + k] = e[k].first;
                s_w[b + k] = e[k].second;
            }
        }
    }
}

extern "C" int gts_build_pages(uint64_t n, uint64_t m, const uint64_t* row_ptr, const uint32_t* col_idx,
                               const uint32_t* weights, const gts_page_config* cfg, gts_graph** out) {
    clear_error();
    if (!row_ptr || !out || (m > 0 && !col_idx)) return fail(GTS_EINVAL, "NULL argument");
    *out = nullptr;
    // struct_size: 16 = the 1.0 layout (no owner fields), sizeof = current; 0 = current
    gts_page_config pc;
    std::memset(&pc, 0, sizeof(pc));
    if (cfg) {
        const uint32_t sz = cfg->struct_size ? cfg->struct_size : (uint32_t)sizeof(gts_page_config);
        if (sz < 16) return fail(GTS_EINVAL, "gts_page_config.struct_size too small");
        std::memcpy(&pc, cfg, std::min<size_t>(sz, sizeof(pc)));
    }
    if (n == 0) return fail(GTS_EINVAL, "n must be >= 1");
    if (n >= (1ull << 32)) return fail(GTS_EOVERFLOW, "n >= 2^32 (u32 VIDs; 0xFFFFFFFF is the NULL/empty sentinel)");
    uint32_t pb = pc.page_bytes ? pc.page_bytes : kDefaultPageBytes;
    uint32_t enc = pc.entry_encoding;
    if (!valid_page_bytes(pb)) return fail(GTS_EINVAL, "page_bytes %u must be a power of two in [256, 2^30]", pb);
    if (enc > GTS_ENTRY_PID16_SLOT16) return fail(GTS_EINVAL, "unknown entry encoding %u", enc);
    if (row_ptr[0] != 0 || row_ptr[n] != m) return fail(GTS_EINVAL, "row_ptr[0] must be 0 and row_ptr[n] == m");
    bool bad_row = false;
    #pragma omp parallel for reduction(||:bad_row)
    for (int64_t v = 0; v < (int64_t)n; ++v) bad_row = bad_row || (row_ptr[v + 1] < row_ptr[v]);
    if (bad_row) return fail(GTS_EINVAL, "row_ptr is not monotone");
    bool bad_col = false;
    #pragma omp parallel for reduction(||:bad_col)
    for (int64_t k = 0; k < (int64_t)m; ++k) bad_col = bad_col || (col_idx[k] >= n);
    if (bad_col) return fail(GTS_EINVAL, "col_idx has an entry >= n");

    const uint32_t known = GTS_BUILD_DEGREE_ORDER | GTS_BUILD_SYMMETRIC | GTS_BUILD_OWNER_FILTER;
    if (pc.flags & ~known) return fail(GTS_EINVAL, "unknown page_config flags 0x%x", pc.flags);
    const bool weighted = weights != nullptr;
    const bool ordered = pc.flags & GTS_BUILD_DEGREE_ORDER;
    const bool symmetric = pc.flags & GTS_BUILD_SYMMETRIC;
    const bool filtered = pc.flags & GTS_BUILD_OWNER_FILTER;
    if (filtered) {
        if (pc.owner_world < 1 || pc.owner_rank >= pc.owner_world)
            return fail(GTS_EINVAL, "owner filter: rank %u of world %u", pc.owner_rank, pc.owner_world);
        if (pc.owner_strategy > GTS_STRATEGY_S_BCAST) return fail(GTS_EINVAL, "owner filter: unknown strategy");
    }
    std::vector<uint64_t> s_row;
    std::vector<uint32_t> s_col, s_w;
    if (symmetric) {
        symmetrise(n, row_ptr, col_idx, weights, s_row, s_col, s_w);
        row_ptr = s_row.data();
        col_idx = s_col.data();
        if (weighted) weights = s_w.data();
        m = 2 * m;
    }
    // Degree ordering (GTS_BUILD_DEGREE_ORDER): rename vertices by descending
    // in-degree (ties by VID) and build the pages of the renamed graph.
    std::vector<uint32_t> new_of_old, old_of_new;
    std::vector<uint64_t> o_row;
    std::vector<uint32_t> o_col, o_w;
    if (ordered) {
        std::vector<uint32_t> indeg(n, 0);
        #pragma omp parallel for schedule(static, 1 << 16)
        for (int64_t k = 0; k < (int64_t)m; ++k) __atomic_fetch_add(&indeg[col_idx[k]], 1u, __ATOMIC_RELAXED);
        uint32_t maxd = 0;
        for (uint64_t v = 0; v < n; ++v) maxd = std::max(maxd, indeg[v]);
        std::vector<uint64_t> bucket((size_t)maxd + 2, 0);
        for (uint64_t v = 0; v < n; ++v) bucket[maxd - indeg[v] + 1]++;
        for (size_t b = 1; b < bucket.size(); ++b) bucket[b] += bucket[b - 1];
        new_of_old.resize(n);
        old_of_new.resize(n);
        for (uint64_t v = 0; v < n; ++v) {
            uint32_t id = (uint32_t)(bucket[maxd - indeg[v]]++);
            new_of_old[v] = id;
            old_of_new[id] = (uint32_t)v;
        }
        std::vector<uint32_t>().swap(indeg);
        o_row.resize(n + 1);
        o_row[0] = 0;
        for (uint64_t i = 0; i < n; ++i) o_row[i + 1] = o_row[i] + (row_ptr[old_of_new[i] + 1] - row_ptr[old_of_new[i]]);
        o_col.resize(m);
        if (weighted) o_w.resize(m);
        #pragma omp parallel for schedule(dynamic, 1024)
        for (int64_t i = 0; i < (int64_t)n; ++i) {
            const uint64_t src = row_ptr[old_of_new[i]], b = o_row[i], len = o_row[i + 1] - b;
            if (!weighted) {
                for (uint64_t k = 0; k < len; ++k) o_col[b + k] = new_of_old[col_idx[src + k]];
                std::sort(o_col.begin() + b, o_col.begin() + b + len);
            } else {
                std::vector<std::pair<uint32_t, uint32_t>> e(len);
                for (uint64_t k = 0; k < len; ++k) e[k] = {new_of_old[col_idx[src + k]], weights[src + k]};
                std::sort(e.begin(), e.end());
                for (uint64_t k = 0; k < len; ++k) {
                    o_col[b + k] = e[k].first;
                    o_w[b + k] = e[k].second;
                }
            }
        }
        row_ptr = o_row.data();
        col_idx = o_col.data();
        if (weighted) weights = o_w.data();
    }
    std::vector<PagePlanEntry> plan;
    gts_graph_stats st;
    int rc = plan_pages(n, row_ptr, weighted, pb, enc, plan, &st);
    if (rc) return rc;

    gts_graph* g = new (std::nothrow) gts_graph();
    if (!g) return fail(GTS_ENOMEM, "graph alloc");
    g->n = n;
    g->m = m;
    g->page_bytes = pb;
    g->entry_encoding = enc;
    g->weighted = weighted;
    g->num_pages = plan.size();
    g->n_sp = st.n_sp;
    g->n_lp = st.n_lp;
    g->n_lp_vertices = st.n_lp_vertices;
    g->used_bytes = st.used_bytes;
    g->max_outdeg = st.max_outdeg;
    g->uid = g_next_uid.fetch_add(1);
    g->symmetric = symmetric;
    g->start_vid.resize(g->num_pages);
    g->nslots.resize(g->num_pages);
    g->kind.resize(g->num_pages);
    g->lp_first.resize(g->num_pages);
    g->lp_last.resize(g->num_pages);
    for (uint64_t p = 0; p < g->num_pages; ++p) {
        g->start_vid[p] = plan[p].start_vid;
        g->nslots[p] = plan[p].nslots;
        g->kind[p] = plan[p].kind;
        g->lp_first[p] = plan[p].lp_first;
        g->lp_last[p] = plan[p].lp_last;
    }
    // the pages this graph holds: all, or (owner filter) the pages of one rank
    std::vector<uint32_t> held;
    if (filtered && pc.owner_strategy != GTS_STRATEGY_S_BCAST && pc.owner_world > 1) {
        std::vector<int32_t> owner;
        std::vector<uint64_t> vr;
        partition(g, pc.owner_strategy, (int)pc.owner_world, owner, vr);
        g->host_loc.assign(g->num_pages, UINT32_MAX);
        for (uint64_t p = 0; p < g->num_pages; ++p)
            if (owner[p] == (int32_t)pc.owner_rank) {
                g->host_loc[p] = (uint32_t)held.size();
                held.push_back((uint32_t)p);
            }
    }
    if (filtered) {
        g->owner_rank = (int32_t)pc.owner_rank;
        g->owner_world = pc.owner_world;
        g->owner_strategy = pc.owner_strategy;
    }
    g->n_host_pages = g->host_loc.empty() ? g->num_pages : held.size();
    g->pages_alloc = (size_t)g->n_host_pages * pb;
    size_t alloc = (g->pages_alloc + 4095) & ~(size_t)4095;
    if (alloc == 0) alloc = 4096;
    g->pages = (uint8_t*)std::aligned_alloc(4096, alloc);
    if (!g->pages) { delete g; return fail(GTS_ENOMEM, "cannot allocate %zu bytes of pages", alloc); }

    // PID16_SLOT16: physical ID of every vertex = (first page holding it, slot)
    std::vector<uint32_t> phys;
    if (enc == GTS_ENTRY_PID16_SLOT16) {
        phys.resize(n);
        for (uint64_t p = 0; p < g->num_pages; ++p) {
            if (plan[p].kind == GTS_PAGE_LP) {
                if (plan[p].lp_first == (int64_t)p) phys[plan[p].start_vid] = (uint32_t)(p << 16);
            } else {
                for (uint32_t s = 0; s < plan[p].nslots; ++s) phys[plan[p].start_vid + s] = (uint32_t)(p << 16) | s;
            }
        }
    }
    const uint64_t wpe = rec_edge_words(weighted), hdrb = 4 * rec_hdr_words(weighted);
    const uint64_t lp_cap = (pb - kLpFooter - kSlotBytes - hdrb) / (4 * wpe);

    #pragma omp parallel for schedule(dynamic, 4)
    for (int64_t hp = 0; hp < (int64_t)g->n_host_pages; ++hp) {
        const int64_t p = g->host_loc.empty() ? hp : (int64_t)held[hp];
        uint8_t* pg = g->pages + (size_t)hp * pb;
        std::memset(pg, 0, pb);
        const PagePlanEntry& e = plan[p];
        // entries after the record header: adj[len], or (adj, w) pairs for weighted records
        auto put_entries = [&](uint8_t* dst, uint64_t k0, uint64_t len) {
            for (uint64_t i = 0; i < len; ++i) {
                uint32_t v = col_idx[k0 + i];
                wr32(dst + 4 * wpe * i, enc == GTS_ENTRY_PID16_SLOT16 ? phys[v] : v);
                if (weighted) wr32(dst + 8 * i + 4, weights[k0 + i]);
            }
        };
        if (e.kind == GTS_PAGE_LP) {
            uint64_t v = e.start_vid;
            uint64_t deg = row_ptr[v + 1] - row_ptr[v];
            uint64_t c = (uint64_t)(p - e.lp_first);
            uint64_t k0 = c * lp_cap, len = std::min(lp_cap, deg - k0);
            wr32(pg, (uint32_t)len);
            put_entries(pg + hdrb, row_ptr[v] + k0, len);
            uint8_t* end = pg + pb;
            wr32(end - 4, GTS_PAGE_LP);
            wr32(end - 8, 1);
            wr32(end - 12, (uint32_t)c);
            wr32(end - 16, (uint32_t)deg);
            wr32(end - kLpFooter - 8, (uint32_t)v);
            wr32(end - kLpFooter - 4, 0);
        } else {
            uint8_t* end = pg + pb;
            uint64_t off = 0;
            for (uint32_t s = 0; s < e.nslots; ++s) {
                uint64_t v = (uint64_t)e.start_vid + s;
                uint64_t deg = row_ptr[v + 1] - row_ptr[v];
                wr32(pg + off, (uint32_t)deg);
                put_entries(pg + off + hdrb, row_ptr[v], deg);
                uint8_t* slot = end - kSpFooter - kSlotBytes * (uint64_t)(s + 1);
                wr32(slot, (uint32_t)v);
                wr32(slot + 4, (uint32_t)off);
                off += hdrb + 4 * wpe * deg;
            }
            wr32(end - 4, GTS_PAGE_SP);
            wr32(end - 8, e.nslots);
        }
    }
    build_hot_table(*g, col_idx);
    if (ordered) {
        g->ordered = true;
        g->new_of_old = std::move(new_of_old);
        g->old_of_new = std::move(old_of_new);
    }
    *out = g;
    return GTS_OK;
}

extern "C" int gts_graph_get_stats(const gts_graph* g, gts_graph_stats* out) {
    clear_error();
    if (!g || !out) return fail(GTS_EINVAL, "NULL argument");
    std::memset(out, 0, sizeof(*out));
    out->n = g->n;
    out->m = g->m;
    out->num_pages = g->num_pages;
    out->n_sp = g->n_sp;
    out->n_lp = g->n_lp;
    out->n_lp_vertices = g->n_lp_vertices;
    out->page_bytes = g->page_bytes;
    out->topo_bytes = g->num_pages * (uint64_t)g->page_bytes;
    out->used_bytes = g->used_bytes;
    out->max_outdeg = g->max_outdeg;
    out->weighted = g->weighted ? 1 : 0;
    out->entry_encoding = g->entry_encoding;
    out->n_hot = g->ordered ? (uint32_t)std::min<uint64_t>(g->n, kHotDense) : g->n_hot;
    out->ordered = g->ordered ? 1 : 0;
    out->host_page_bytes = g->n_host_pages * (uint64_t)g->page_bytes;
    out->symmetric = g->symmetric ? 1 : 0;
    out->owner_rank = g->owner_rank;
    out->owner_world = g->owner_world;
    out->owner_strategy = g->owner_strategy;
    return GTS_OK;
}

extern "C" const uint8_t* gts_graph_pages(const gts_graph* g) { return g ? g->pages : nullptr; }

extern "C" int gts_graph_directory(const gts_graph* g, uint32_t* start_vid, uint32_t* nslots, uint32_t* kind,
                                   int64_t* lp_first, int64_t* lp_last) {
    clear_error();
    if (!g) return fail(GTS_EINVAL, "NULL graph");
    size_t P = g->num_pages;
    if (start_vid) std::memcpy(start_vid, g->start_vid.data(), P * 4);
    if (nslots) std::memcpy(nslots, g->nslots.data(), P * 4);
    if (kind) std::memcpy(kind, g->kind.data(), P * 4);
    if (lp_first) std::memcpy(lp_first, g->lp_first.data(), P * 8);
    if (lp_last) std::memcpy(lp_last, g->lp_last.data(), P * 8);
    return GTS_OK;
}

extern "C" int gts_graph_order(const gts_graph* g, uint32_t* internal_of) {
    clear_error();
    if (!g || !internal_of) return fail(GTS_EINVAL, "NULL argument");
    if (g->ordered) std::memcpy(internal_of, g->new_of_old.data(), g->n * 4);
    else
        for (uint64_t v = 0; v < g->n; ++v) internal_of[v] = (uint32_t)v;
    return GTS_OK;
}
