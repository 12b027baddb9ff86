// Weakly connected components over slotted pages (R12).
//
// Paper: "connected components" is a PageRank-like algorithm run by GTS
// (P:308), i.e. whole-topology sweeps (ALL_PAGES, Alg 1 line 7); no
// kernel is given.  B200 design: one sweep over all pages hooks every edge
// into a concurrent union-find forest whose roots are component minima
// (ECL-CC-style hooking with atomicCAS, path halving), then a finalize pass
// points every vertex at its root = the minimum VID of its weakly connected
// component.  One sweep is exact on one GPU.  Strategy-P with N > 1: each
// rank hooks its own pages, labels are merged with an all-reduce(min), and
// the sweep repeats from the merged labels until no rank hooks anything.
// S_BCAST: every rank hooks every page (replicated, exact after one sweep).
// Strategy-S: routed label propagation on symmetrised pages (traverse.cu).
#include <cuda_runtime.h>
#include <nccl.h>

#include <cstdlib>
#include <cstring>

#include "comm.h"
#include "expand.cuh"
#include "sweep.cuh"
#include "traverse.h"

namespace gts {

// Union-find over the page sweep (ECL-CC style hooking).  Invariant:
// parent[v] <= v, roots satisfy parent[r] = r, and a hook always points the
// larger root at the smaller one, so the root of every component is its
// minimum (internal) VID.  One sweep over all pages hooks every edge; a
// finalize pass then points every vertex at its root.  Path halving in find
// writes only ancestors, so concurrent finds/hooks are benign.
__device__ __forceinline__ uint32_t uf_find(uint32_t* parent, uint32_t x) {
    uint32_t cur = __ldcg(parent + x);
    if (cur != x) {
        uint32_t prev = x, next;
        while (cur > (next = __ldcg(parent + cur))) {
            parent[prev] = next;
            prev = cur;
            cur = next;
        }
    }
    return cur;
}

__device__ __forceinline__ bool uf_hook(uint32_t* parent, uint32_t a, uint32_t b) {
    uint32_t ra = uf_find(parent, a), rb = uf_find(parent, b);
    bool hooked = false;
    while (ra != rb) {
        if (ra < rb) {
            const uint32_t ret = atomicCAS(parent + rb, rb, ra);
            if (ret == rb) { hooked = true; break; }
            rb = ret;
        } else {
            const uint32_t ret = atomicCAS(parent + ra, ra, rb);
            if (ret == ra) { hooked = true; break; }
            ra = ret;
        }
    }
    return hooked;
}

// Per edge u -> v: the payload is parent[u] read once per vertex per tile; if
// parent[v] equals it the endpoints already share a tree (trees only ever
// merge, so equal pointers, even stale ones, mean one component) and the edge
// costs a single gather; otherwise a full hook.  After the sampling pass below
// most vertices point straight at their component's root, so most edges of
// the giant component end here.
//
// Giant filter: after the sampling pass, gbm marks the vertices whose parent
// was the root r* of vertex 0's tree (on degree-ordered pages the giant
// component); an edge whose source points at r* and whose destination bit is
// set is skipped on a bitmap test (n/8 bytes, L1/L2-resident like BFS's
// visited bitmap) without touching parent[].
//
// Plain walk (expand.cuh dense_tile_plain): in a tile whose vertices with edges all have
// their gbm bit set (parent = r* for good: r* = parent[0] = 0 is the smallest VID, so it
// stays a root), every edge u -> v is the edge r* -> v, so no owner is needed; words
// below the all-giant prefix gfloor (destinations already in r*'s tree) are skipped.
template <bool W>
struct WccOp {
    static constexpr bool kReadWeights = false;
    static constexpr bool kWeighted = W;
    static constexpr bool kFastDense = !W;
    uint32_t* parent;
    bool changed;
    const uint32_t* gbm;      // nullptr: no giant filter
    uint32_t rstar;
    uint32_t gfloor;          // all-giant prefix (vertices); 0 = no plain walk
    uint32_t plain8;
    uint32_t plan_floor;
    __device__ uint32_t fast_floor() const { return gbm ? gfloor : 0u; }
    __device__ bool done(uint32_t v) const { return test_bit(gbm, v); }
    __device__ uint32_t plain_src() const { return rstar; }
    __device__ void plain_edges(uint32_t) {}
    __device__ const uint32_t* frontier() const { return nullptr; }
    __device__ bool select(uint32_t) { return true; }
    __device__ uint32_t payload(uint32_t v, uint32_t) { return __ldcg(parent + v); }
    __device__ bool select_lp(uint32_t vid, uint32_t, uint32_t, uint32_t& pl) {
        pl = __ldcg(parent + vid);
        return true;
    }
    __device__ __forceinline__ void edges(const uint32_t* dst, const uint32_t*, const uint32_t* pl,
                                          const uint32_t* src, const bool* valid) {
        bool live[kEdgesPerThread];
#pragma unroll
        for (int q = 0; q < kEdgesPerThread; ++q) {
            live[q] = valid[q];
            if (gbm && valid[q] && pl[q] == rstar) live[q] = !((__ldg(gbm + (dst[q] >> 5)) >> (dst[q] & 31)) & 1u);
        }
        uint32_t pv[kEdgesPerThread];
#pragma unroll
        for (int q = 0; q < kEdgesPerThread; ++q) pv[q] = live[q] ? __ldcg(parent + dst[q]) : 0u;
#pragma unroll
        for (int q = 0; q < kEdgesPerThread; ++q)
            if (live[q] && pv[q] != pl[q] && src[q] != dst[q] && uf_hook(parent, src[q], dst[q])) changed = true;
    }
    __device__ void end_page() {}
};

// Sampling pass (Afforest-style, Sutton et al. 2018, adapted to out-edge
// pages): every vertex hooks only its first `ks` out-neighbours (an LP vertex:
// from its first chunk).  Rows are sorted by destination, so on degree-ordered
// pages these are the vertex's highest in-degree neighbours and the giant
// component's trees form almost at once.  The full sweep that follows still
// visits every edge (the result is exact); the sample only makes its edges
// cheap (one gather instead of two finds).
__global__ void __launch_bounds__(kThreads, 2)
wcc_sample_kernel(PageSet ps, uint32_t* parent, uint32_t* work_ctr, uint32_t ks, int weighted) {
    const uint32_t hdr = rec_hdr_words(weighted != 0), ew = rec_edge_words(weighted != 0);
    __shared__ uint32_t s_item;
    const int tid = threadIdx.x;
    const uint64_t pol = policy_evict_first();
    for (;;) {
        if (tid == 0) s_item = atomicAdd(work_ctr, 1u);
        __syncthreads();
        const uint32_t it = s_item;
        __syncthreads();
        if (it >= ps.count) break;
        uint32_t pid;
        const uint8_t* data;
        page_at(ps, it, pid, data);
        const uint8_t* end = data + ps.page_bytes;
        const uint32_t kind = ld32(end - 4);
        const uint32_t* words = reinterpret_cast<const uint32_t*>(data);
        if (kind == GTS_PAGE_LP) {
            const uint32_t vid = ld32(end - kLpFooter - kSlotBytes);
            const uint32_t chunk = ld32(end - 12);
            const uint32_t len = ld32(data);
            if (chunk == 0 && (uint32_t)tid < min(ks, len)) {
                const uint32_t v = decode_entry(ps, ld_stream_u32(words + hdr + ew * tid, pol));
                if (v != vid) uf_hook(parent, vid, v);
            }
        } else {
            const uint32_t nslots = ld32(end - 8);
            const uint32_t start = ld32(end - kSpFooter - kSlotBytes);
            for (uint32_t u = tid; u < nslots; u += kThreads) {
                const uint32_t off = ld_stream_u32(end - kSpFooter - kSlotBytes * (uint64_t)(u + 1) + 4, pol) >> 2;
                const uint32_t deg = ld_stream_u32(words + off, pol);
                const uint32_t kk = min(ks, deg);
                for (uint32_t k = 0; k < kk; ++k) {
                    const uint32_t v = decode_entry(ps, ld_stream_u32(words + off + hdr + ew * k, pol));
                    if (v != start + u) uf_hook(parent, start + u, v);
                }
            }
        }
    }
}

template <bool W, int MB = 2>
__global__ void __launch_bounds__(kThreads, MB)
wcc_sweep_kernel(PageSet ps, uint32_t* parent, uint32_t* work_ctr, uint32_t* changed, const uint32_t* gbm,
                 const uint32_t* rstar, uint32_t plain8, uint32_t wcc_plan_floor) {
    __shared__ TileSmem sm;
    // rstar[1] = first gbm word that is not all ones (wcc_giant_kernel)
    const uint32_t gfloor = gbm && plain8 <= 8 ? (uint32_t)min((uint64_t)__ldg(rstar + 1) * 32, (uint64_t)0xFFFFFFFFu) : 0u;
    WccOp<W> op{parent, false, gbm, gbm ? __ldg(rstar) : 0u, gfloor, plain8, wcc_plan_floor};
    expand_pages(ps, op, sm, work_ctr);
    if (__syncthreads_or(op.changed) && threadIdx.x == 0) *changed = 1u;
}

__global__ void wcc_init_kernel(uint32_t* label, uint64_t n) {
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) label[i] = (uint32_t)i;
}

// gbm bit v = (parent[v] == parent[0]); rstar[0] = parent[0]; rstar[1] = the first gbm
// word that is not all ones (rstar[1] must be 0xFFFFFFFF on entry; run after a finalize pass)
__global__ void wcc_giant_kernel(const uint32_t* parent, uint64_t n, uint32_t* gbm, uint32_t* rstar) {
    const uint32_t r = __ldcg(parent);
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    const uint64_t nw = (n + 31) / 32 * 32;
    uint32_t hole = 0xFFFFFFFFu;
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nw; i += stride) {
        const bool in = i < n && __ldcg(parent + i) == r;
        const uint32_t b = __ballot_sync(0xFFFFFFFFu, in);
        if ((threadIdx.x & 31) == 0) gbm[i >> 5] = b;
        if (b != 0xFFFFFFFFu) hole = min(hole, (uint32_t)(i >> 5));
    }
    if ((threadIdx.x & 31) == 0 && hole != 0xFFFFFFFFu) atomicMin(rstar + 1, hole);
    if (blockIdx.x == 0 && threadIdx.x == 0) *rstar = r;
}

// every vertex points at its root (the component's minimum VID)
// Four consecutive vertices per thread per step, their root walks interleaved
// so four pointer-chasing reads are in flight (one per vertex per hop).
__global__ void wcc_finalize_kernel(uint32_t* parent, uint64_t n) {
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    const uint64_t t = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const uint64_t n4 = n >> 2;
    uint4* p4 = reinterpret_cast<uint4*>(parent);
    for (uint64_t q = t; q < n4; q += stride) {
        const uint4 v = __ldcg(p4 + q);
        uint32_t r[4] = {v.x, v.y, v.z, v.w};
        bool more = true;
        while (more) {
            uint32_t p[4];
#pragma unroll
            for (int k = 0; k < 4; ++k) p[k] = __ldcg(parent + r[k]);
            more = false;
#pragma unroll
            for (int k = 0; k < 4; ++k) {
                more |= p[k] != r[k];
                r[k] = p[k];
            }
        }
        p4[q] = make_uint4(r[0], r[1], r[2], r[3]);
    }
    for (uint64_t i = 4 * n4 + t; i < n; i += stride) {
        uint32_t r = __ldcg(parent + i);
        while (r != __ldcg(parent + r)) r = __ldcg(parent + r);
        parent[i] = r;
    }
}

enum { kBufLabel = 30, kBufWccCtr, kBufWccGiant };
constexpr int kBufWccMulti = 400;   // multi-rank slot i: kBufWccMulti + 4 i + k

}  // namespace gts

using namespace gts;

extern "C" int gts_wcc(gts_context* c, const gts_graph* g, const gts_run_config* cfg, uint32_t* label_out,
                       gts_run_stats* st) {
    clear_error();
    const double t_start = now_s();
    gts_run_config rc;
    GTS_TRY(validate_common(c, g, cfg, &rc));
    if (rc.flags & GTS_MICRO_MASK) return fail(GTS_EUNSUPPORTED, "GTS_MICRO_* techniques apply to gts_bfs and gts_pagerank");
    if (!label_out) return fail(GTS_EINVAL, "NULL output");
    Ranks R;
    GTS_TRY(make_ranks(c, rc, &R));
    const uint64_t n = g->n;
    const int N = R.world, L = R.nloc;
    const uint32_t strat = N > 1 ? rc.strategy : GTS_STRATEGY_P;
    const bool streamed = choose_streamed(c, g, rc, strat == GTS_STRATEGY_S ? 4 * n / N + n / 8 : 4 * n);
    double upload_s = 0;
    GTS_TRY(ensure_graph(c, g, rc.strategy, !streamed, &upload_s));
    // Strategy-S: routed min-label propagation on symmetrised pages (traverse.cu)
    if (strat == GTS_STRATEGY_S) return traverse_multi(c, g, 0, rc, R, label_out, st, kWCCLP, t_start, streamed, upload_s);
    // One rank, Strategy-P (each rank hooks its pages; forests merged by all-reduce(min), repeated
    // until no rank hooks) or S_BCAST (every rank hooks every page: exact after one sweep, no exchange)
    const bool timing = rc.flags & GTS_RUN_TIMING;
    cudaStream_t s = c->stream;
    const int eg = c->num_sms * 4;
    std::vector<int32_t> owner;
    std::vector<uint64_t> vr;
    partition(g, strat, N, owner, vr);
    std::vector<uint32_t*> label(L), ctr(L);
    std::vector<std::vector<uint32_t>> pages(L);
    std::vector<const uint32_t*> d_pages(L);
    for (int i = 0; i < L; ++i) {
        if (R.virt) {
            for (uint64_t j = 0; j < g->num_pages; ++j)
                if (strat == GTS_STRATEGY_S_BCAST || owner[j] == R.rank(i)) pages[i].push_back((uint32_t)j);
            uint32_t* dp;
            GTS_TRY(c->buf(kBufWccMulti + 4 * i, std::max<size_t>(pages[i].size(), 1) * 4, (void**)&dp));
            if (!pages[i].empty())
                GTS_CUDA(cudaMemcpyAsync(dp, pages[i].data(), pages[i].size() * 4, cudaMemcpyHostToDevice, s));
            d_pages[i] = dp;
        } else {
            pages[i] = c->dg.h_local_list;
            d_pages[i] = (c->dg.all_local && !streamed) ? nullptr : c->dg.local_list;
        }
        GTS_TRY(c->buf(L == 1 ? kBufLabel : kBufWccMulti + 4 * i + 1, n * 4, (void**)&label[i]));
        GTS_TRY(c->buf(L == 1 ? kBufWccCtr : kBufWccMulti + 4 * i + 2, 8, (void**)&ctr[i]));
        wcc_init_kernel<<<eg, 256, 0, s>>>(label[i], n);
    }
    GTS_CUDA(cudaGetLastError());
    // three 512-thread CTAs per SM for the sweep (40 registers; RMAT-27 sweep 17.4 -> 14.6 ms
    // against two: the third CTA covers the per-tile barriers)
    auto sweep_k = g->weighted ? wcc_sweep_kernel<true, 3> : wcc_sweep_kernel<false, 3>;
    // plain walk of all-giant tiles (WccOp): every tile qualifies by its selected edges
    // (WCC selects every vertex); RMAT-27 WCC kernels 12.60 -> 10.83 ms
    // (degree-ordered pages only: in natural VID order the all-giant prefix is a few
    // vertices, no tile qualifies, and the plan would be pure overhead; 9 = off)
    const uint32_t wcc_plain8 = g->ordered ? 0u : 9u;
    // whole-page plans (expand.cuh plan_plain_tiles): runs of all-giant tiles streamed as one
    // range; RMAT-27 WCC kernels 9.90 ms against 10.84 deciding per tile
    constexpr uint32_t wcc_plan_floor = 0u;
    int grid = 0;
    GTS_TRY(sms_grid(c, (const void*)sweep_k, kThreads, 0, &grid));
    uint64_t launches = L, main_launches = 0;
    uint32_t sweeps = 0;
    uint32_t* hs = (uint32_t*)c->h_small;
    SweepStats ss;
    // sampling pass + compression (one rank, resident pages only: streamed, it would cost a
    // whole extra transfer of the topology); gts_run_config.wcc_sample = k neighbours
    const uint32_t ks = rc.wcc_sample == GTS_OFF ? 0u : rc.wcc_sample ? rc.wcc_sample : 1u;
    // persisting-L2 window on the head of the union-find forest (degree-ordered pages: the
    // most probed parents); gts_run_config.l2_persist_mib
    bool persist = false;
    if (!streamed && g->ordered && N == 1) {
        const size_t want = std::min<size_t>(l2_persist_mib(rc) << 20, n * 4);
        if (want > 0) {
            GTS_TRY(persist_window(c, s, label[0], want));
            persist = true;
        }
    }
    uint32_t* gbm = nullptr;   // giant filter bitmap (+ r* after it)
    if (!streamed && ks > 0 && N == 1) {
        std::pair<cudaEvent_t, cudaEvent_t> ev;
        if (timing) { ev = c->t_main.next(); cudaEventRecord(ev.first, s); }
        GTS_CUDA(cudaMemsetAsync(ctr[0], 0, 4, s));
        PageSet ps;
        ps.base = c->dg.pages;
        ps.list = d_pages[0];
        ps.loc = c->dg.loc;
        ps.d_count = nullptr;
        ps.count = c->dg.n_local;
        ps.page_bytes = g->page_bytes;
        ps.mode = c->dg.all_local ? kAddrByPid : kAddrByLoc;
        ps.entry_encoding = g->entry_encoding;
        ps.rvt_start = c->dg.rvt_start;
        int sg = 0;
        GTS_TRY(sms_grid(c, (const void*)wcc_sample_kernel, kThreads, 0, &sg));
        wcc_sample_kernel<<<sg, kThreads, 0, s>>>(ps, label[0], ctr[0], ks, g->weighted ? 1 : 0);
        wcc_finalize_kernel<<<eg, 256, 0, s>>>(label[0], n);
        GTS_TRY(c->buf(kBufWccGiant, (n + 31) / 32 * 4 + 16, (void**)&gbm));
        GTS_CUDA(cudaMemsetAsync(gbm + (n + 31) / 32 + 1, 0xFF, 4, s));
        wcc_giant_kernel<<<eg, 256, 0, s>>>(label[0], n, gbm, gbm + (n + 31) / 32);
        if (timing) cudaEventRecord(ev.second, s);
        GTS_CUDA(cudaGetLastError());
        launches += 2;
    }
    for (;;) {
        for (int i = 0; i < L; ++i) {
            GTS_CUDA(cudaMemsetAsync(ctr[i] + 1, 0, 4, s));
            std::vector<uint32_t> hl(pages[i]);
            GTS_TRY(sweep_pages(c, g, rc, streamed, &hl, d_pages[i], (uint32_t)hl.size(), nullptr,
                                [&](const PageSet& ps, int cap) -> int {
                                    GTS_CUDA(cudaMemsetAsync(ctr[i], 0, 4, s));
                                    std::pair<cudaEvent_t, cudaEvent_t> e2;
                                    if (timing) { e2 = c->t_main.next(); cudaEventRecord(e2.first, s); }
                                    sweep_k<<<std::min(grid, cap), kThreads, 0, s>>>(
                                        ps, label[i], ctr[i], ctr[i] + 1, gbm, gbm ? gbm + (n + 31) / 32 : nullptr,
                                        wcc_plain8, wcc_plan_floor);
                                    if (timing) cudaEventRecord(e2.second, s);
                                    GTS_CUDA(cudaGetLastError());
                                    ++main_launches;
                                    return GTS_OK;
                                }, &ss));
        }
        ++sweeps;
        const bool merge = N > 1 && strat == GTS_STRATEGY_P;
        if (merge) {                    // a12: forests merged by min, hook flags by max
            std::pair<cudaEvent_t, cudaEvent_t> ev;
            if (timing) { ev = c->t_merge.next(); cudaEventRecord(ev.first, s); }
            std::vector<void*> lb(L), fb(L);
            for (int i = 0; i < L; ++i) {
                lb[i] = label[i];
                fb[i] = ctr[i] + 1;
            }
            GTS_TRY(R.allreduce(lb.data(), n, kCU32, kCMin));
            GTS_TRY(R.allreduce(fb.data(), 1, kCU32, kCMax));
            if (timing) cudaEventRecord(ev.second, s);
        }
        std::pair<cudaEvent_t, cudaEvent_t> ev;
        if (timing) { ev = c->t_finish.next(); cudaEventRecord(ev.first, s); }
        for (int i = 0; i < L; ++i) wcc_finalize_kernel<<<eg, 256, 0, s>>>(label[i], n);
        if (timing) cudaEventRecord(ev.second, s);
        launches += L;
        if (!merge) break;              // union-find over every page is exact after one sweep
        GTS_CUDA(cudaMemcpyAsync(hs, ctr[0] + 1, 4, cudaMemcpyDeviceToHost, s));
        GTS_CUDA(cudaStreamSynchronize(s));
        if (hs[0] == 0) break;
    }
    if (persist) GTS_TRY(persist_window(c, s, nullptr, 0));
    GTS_TRY(deliver(c, g, label[0], label_out, rc.out_location, true));
    if (st) {
        std::memset(st, 0, sizeof(*st));
        st->wall_s = now_s() - t_start;
        st->upload_s = upload_s;
        if (timing) {
            st->main_kernel_s = c->t_main.sum_s();
            st->merge_s = c->t_merge.sum_s();
            st->finish_s = c->t_finish.sum_s();
            st->h2d_s = c->t_h2d.sum_s();
        }
        uint64_t np = 0;
        for (auto& p : pages) np += p.size();
        st->pages_processed = np * sweeps;
        st->h2d_bytes = ss.h2d_bytes;
        st->edges_traversed = (strat == GTS_STRATEGY_S_BCAST ? g->m * (uint64_t)L : g->m * (uint64_t)L / (uint64_t)N) *
                              sweeps;
        st->nccl_bytes = R.bytes;
        st->launches = launches + main_launches;
        st->main_kernel_launches = main_launches;
        st->levels_or_iters = sweeps;
        st->wa_bytes = n * 4;
    } else if (timing) {
        c->t_main.sum_s();
        c->t_merge.sum_s();
        c->t_finish.sum_s();
        c->t_h2d.sum_s();
    }
    return GTS_OK;
}
