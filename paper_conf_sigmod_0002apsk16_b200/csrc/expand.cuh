// Generic page expansion for sm_100a, shared by BFS, SSSP and WCC: persistent
// CTAs take whole slotted pages from an atomic page queue; inside a page the
// 16 warps work independently (no CTA barrier between a page's first and last
// vertex).
//
// Paper: K_SP / K_LP (Alg 2-5) give each vertex of an SP to one
// (virtual) warp (VWC) and each ADJLIST entry of an LP to one thread;
// App E proposes choosing edge- or vertex-centric processing per
// page by density.  B200 design:
//  * SP pages are consumed in groups of 32 consecutive slots claimed by warps
//    from a per-page shared counter.  A lane per slot reads the record offset
//    (one coalesced slot read); degrees are offset differences; the frontier
//    test per vertex is folded into __ballot_sync.
//  * Dense group (selected edges >= half of the group's record words, always
//    true for PageRank-like sweeps): the group's record region is streamed with
//    16-byte evict_first loads and each 4-word chunk finds its owner by a
//    5-step binary search over the 33 group offsets in shared memory.
//  * Sparse group: the selected vertices are compacted with __popc of the
//    ballot, their degrees prefix-summed with shuffles, and the warp expands
//    their edges edge-parallel (4 consecutive edges per lane).
//  * LP pages (one vertex, up to 262,137 entries at 1 MiB) are swept by all 16
//    warps of the CTA; a hub spans several LPs and therefore several CTAs.
// Each op receives 4 edges at a time whose adjacency words were loaded back
// to back, and issues its own per-edge loads (visited bits, dist, parents) as
// a batch before acting on them.
#pragma once

#include <cstdint>

#include "memops.cuh"
#include "runtime.h"

namespace gts {

constexpr int kThreads = 512;
constexpr int kWarps = kThreads / 32;
constexpr int kEdgesPerThread = 4;   // one 16-byte group per op call
constexpr int kDenseUnroll = 2;      // 16-byte loads in flight per lane in dense groups

__device__ __forceinline__ uint32_t ld32(const uint8_t* p) { return __ldg(reinterpret_cast<const uint32_t*>(p)); }

__device__ __forceinline__ void page_at(const PageSet& ps, uint32_t i, uint32_t& pid, const uint8_t*& data) {
    pid = ps.list ? __ldg(ps.list + i) : i;
    uint64_t di = ps.mode == kAddrByPid ? pid : (ps.mode == kAddrByLoc ? __ldg(ps.loc + pid) : i);
    data = ps.base + di * (uint64_t)ps.page_bytes;
}

// ADJLIST entry -> VID (App A: VID = RVT[ADJ_PID].START_VID + ADJ_OFF)
__device__ __forceinline__ uint32_t decode_entry(const PageSet& ps, uint32_t e) {
    return ps.entry_encoding == GTS_ENTRY_VID32 ? e : __ldg(ps.rvt_start + (e >> 16)) + (e & 0xFFFFu);
}

__device__ __forceinline__ bool test_bit(const uint32_t* bm, uint32_t v) {
    return (__ldg(bm + (v >> 5)) >> (v & 31)) & 1u;
}

struct WarpSmem {
    uint32_t off[33];      // dense: record word offsets of the group (off[nv] = end of the last record)
    uint32_t pay[32];      // payload of each slot (dense) or of each selected vertex (sparse)
    uint32_t pre[33];      // sparse: exclusive prefix of the selected degrees
    uint32_t eoff[32];     // sparse: word index of the first ADJLIST entry
    uint32_t src[32];      // sparse: VID
    uint32_t deg[32];      // sparse: degree
    uint32_t selmask;      // dense: ballot of the selected slots
};

struct TileSmem {
    WarpSmem w[kWarps];
    uint32_t item;
    uint32_t gctr;         // next 32-slot group of the current page
};

// Op interface:
//   static constexpr bool kReadWeights;  -- the op needs edge weights
//   static constexpr bool kWeighted;     -- the pages carry weights (record = sz, adj[sz], w[sz])
//   bool select(uint32_t vid)                            -- SP vertex expanded?
//   uint32_t payload(uint32_t vid, uint32_t deg)         -- per selected vertex (called once)
//   bool select_lp(uint32_t vid, uint32_t total_deg, uint32_t chunk_len, uint32_t& payload)
//   void edges(const uint32_t dst[4], const uint32_t w[4], const uint32_t pl[4], const uint32_t src[4],
//              const bool valid[4])
//   void end_page()
template <class Op>
__device__ __forceinline__ void expand_group(const PageSet& ps, Op& op, WarpSmem& ws, const uint8_t* data,
                                             const uint8_t* end, uint32_t start, uint32_t nslots, uint32_t g,
                                             uint64_t pol) {
    constexpr uint32_t wsh = Op::kWeighted ? 1 : 0;
    const int lane = threadIdx.x & 31;
    const uint32_t* words = reinterpret_cast<const uint32_t*>(data);
    const uint32_t j = g * 32 + lane;
    const bool valid = j < nslots;
    const uint32_t v = start + j;
    const bool sel = valid && op.select(v);
    const uint32_t mask = __ballot_sync(0xFFFFFFFFu, sel);
    if (!mask) return;
    // record offsets and degrees (offset differences; the page's last record reads its header)
    uint32_t off = 0;
    const uint8_t* slot = end - kSpFooter - kSlotBytes * (uint64_t)(j + 1);
    if (valid) off = ld_stream_u32(slot + 4, pol) >> 2;
    uint32_t nxt = __shfl_down_sync(0xFFFFFFFFu, off, 1);
    const uint32_t last = min(31u, nslots - 1 - g * 32);           // lane of the group's last slot
    if ((uint32_t)lane == last) {
        if (j + 1 < nslots) nxt = ld_stream_u32(slot - kSlotBytes + 4, pol) >> 2;
        else nxt = off + 1 + (ld32(data + 4ull * off) << wsh);
    }
    const uint32_t deg = valid ? (nxt - off - 1) >> wsh : 0u;
    const uint32_t sdeg = sel ? deg : 0u;
    uint32_t incl = sdeg;                                          // warp inclusive scan of selected degrees
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xFFFFFFFFu, incl, o);
        if (lane >= o) incl += y;
    }
    const uint32_t total = __shfl_sync(0xFFFFFFFFu, incl, 31);
    const uint32_t W0 = __shfl_sync(0xFFFFFFFFu, off, 0), W1 = __shfl_sync(0xFFFFFFFFu, nxt, last);
    const uint32_t pay = sel ? op.payload(v, deg) : 0u;
    if (total == 0) return;
    if (2 * total >= W1 - W0) {
        // ---- dense group: stream the record words, act on the selected owners
        ws.off[lane] = off;
        if (lane == 0) {
            ws.off[last + 1] = W1;
            ws.selmask = mask;
        }
        ws.pay[lane] = pay;
        __syncwarp();
        const uint32_t nv = last + 1;
        const uint32_t smask = mask;
        const uint4* q4 = reinterpret_cast<const uint4*>(data);
        const uint32_t qbeg = W0 >> 2, qend = (W1 + 3) >> 2;
        for (uint32_t qb = qbeg + lane; qb < qend; qb += 32 * kDenseUnroll) {
            uint4 vv[kDenseUnroll];
#pragma unroll
            for (int u = 0; u < kDenseUnroll; ++u) {
                const uint32_t q = qb + 32 * u;
                if (q < qend) vv[u] = ld_stream_v4(q4 + q, pol);
            }
#pragma unroll
            for (int u = 0; u < kDenseUnroll; ++u) {
                const uint32_t q = qb + 32 * u;
                if (q >= qend) break;
                const uint32_t w0 = 4 * q;
                uint32_t lo = 0, hi = nv;                          // off[lo] <= max(w0, W0) < off[hi]
                while (hi - lo > 1) {
                    const uint32_t mid = (lo + hi) >> 1;
                    if (ws.off[mid] <= w0) lo = mid; else hi = mid;
                }
                uint32_t k_ = lo, cur = ws.off[lo], nx = ws.off[lo + 1];
                uint32_t dst[4], wt[4], pl[4], src[4];
                bool ok[4];
#pragma unroll
                for (int k = 0; k < 4; ++k) {
                    const uint32_t w = w0 + k;
                    bool e = w >= W0 && w < W1;
                    if (e) {
                        while (w >= nx) {
                            ++k_;
                            cur = nx;
                            nx = ws.off[k_ + 1];
                        }
                        const uint32_t rel = w - cur, dj = (nx - cur - 1) >> wsh;
                        e = rel >= 1 && rel <= dj && ((smask >> k_) & 1u);
                        wt[k] = (Op::kReadWeights && e) ? ld_stream_l1_u32(words + w + dj, pol) : 0u;
                    } else {
                        wt[k] = 0u;
                    }
                    ok[k] = e;
                    dst[k] = decode_entry(ps, word_of(vv[u], k));
                    pl[k] = ws.pay[k_];
                    src[k] = start + g * 32 + k_;
                }
                op.edges(dst, wt, pl, src, ok);
            }
        }
        __syncwarp();
        return;
    }
    // ---- sparse group: compacted selected vertices, edge-parallel gather
    const uint32_t pos = __popc(mask & ((1u << lane) - 1u));
    const uint32_t nf = __popc(mask);
    if (sel) {
        ws.eoff[pos] = off + 1;
        ws.deg[pos] = deg;
        ws.src[pos] = v;
        ws.pay[pos] = pay;
        ws.pre[pos] = incl - sdeg;
    }
    if (lane == 0) ws.pre[nf] = total;
    __syncwarp();
    for (uint32_t e0 = (uint32_t)lane * 4; e0 < total; e0 += 128) {
        uint32_t lo = 0, hi = nf;                                  // pre[lo] <= e0 < pre[hi]
        while (hi - lo > 1) {
            const uint32_t mid = (lo + hi) >> 1;
            if (ws.pre[mid] <= e0) lo = mid; else hi = mid;
        }
        uint32_t k_ = lo, nx = ws.pre[lo + 1];
        uint32_t dst[4], wt[4], pl[4], src[4];
        bool ok[4];
#pragma unroll
        for (int q = 0; q < 4; ++q) {
            const uint32_t e = e0 + q;
            ok[q] = e < total;
            if (ok[q]) {
                while (e >= nx) nx = ws.pre[++k_ + 1];
            }
            const uint32_t local = e - ws.pre[k_];
            const uint32_t* adj = words + ws.eoff[k_];
            dst[q] = ok[q] ? ld_stream_l1_u32(adj + local, pol) : 0u;
            wt[q] = (Op::kReadWeights && ok[q]) ? ld_stream_l1_u32(adj + ws.deg[k_] + local, pol) : 0u;
            pl[q] = ws.pay[k_];
            src[q] = ws.src[k_];
        }
#pragma unroll
        for (int q = 0; q < 4; ++q) dst[q] = decode_entry(ps, dst[q]);
        op.edges(dst, wt, pl, src, ok);
    }
    __syncwarp();
}

template <class Op>
__device__ void expand_pages(const PageSet& ps, Op& op, TileSmem& sm, uint32_t* work_ctr) {
    const uint32_t count = ps.d_count ? *(volatile const uint32_t*)ps.d_count : ps.count;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const uint64_t pol = policy_evict_first();
    WarpSmem& ws = sm.w[warp];
    for (;;) {
        if (tid == 0) {
            sm.item = atomicAdd(work_ctr, 1u);
            sm.gctr = 0;
        }
        __syncthreads();
        const uint32_t i = sm.item;
        if (i >= count) break;
        uint32_t pid;
        const uint8_t* data;
        page_at(ps, i, pid, data);
        const uint8_t* end = data + ps.page_bytes;
        const uint32_t kind = ld32(end - 4);
        const uint32_t nslots = ld32(end - 8);
        const uint32_t* words = reinterpret_cast<const uint32_t*>(data);
        if (kind == GTS_PAGE_LP) {
            const uint32_t vid = ld32(end - kLpFooter - kSlotBytes);
            const uint32_t total = ld32(end - 16);
            const uint32_t len = ld32(data);
            uint32_t payload = 0;
            if (op.select_lp(vid, total, len, payload)) {
                const uint32_t* adj = words + 1;
                for (uint32_t k0 = tid; k0 < len; k0 += kThreads * kEdgesPerThread) {
                    uint32_t dst[kEdgesPerThread], w[kEdgesPerThread], pl[kEdgesPerThread], src[kEdgesPerThread];
                    bool valid[kEdgesPerThread];
#pragma unroll
                    for (int q = 0; q < kEdgesPerThread; ++q) {
                        const uint32_t k = k0 + q * kThreads;
                        valid[q] = k < len;
                        dst[q] = valid[q] ? ld_stream_u32(adj + k, pol) : 0u;
                        w[q] = (Op::kReadWeights && valid[q]) ? ld_stream_u32(adj + len + k, pol) : 0u;
                        pl[q] = payload;
                        src[q] = vid;
                    }
#pragma unroll
                    for (int q = 0; q < kEdgesPerThread; ++q) dst[q] = decode_entry(ps, dst[q]);
                    op.edges(dst, w, pl, src, valid);
                }
            }
        } else {
            const uint32_t start = ld32(end - kSpFooter - kSlotBytes);
            const uint32_t ngroups = (nslots + 31) >> 5;
            for (;;) {
                uint32_t g = 0;
                if (lane == 0) g = atomicAdd(&sm.gctr, 1u);
                g = __shfl_sync(0xFFFFFFFFu, g, 0);
                if (g >= ngroups) break;
                expand_group(ps, op, ws, data, end, start, nslots, g, pol);
            }
        }
        op.end_page();
        __syncthreads();                      // sm.item / sm.gctr are rewritten for the next page
    }
}

}  // namespace gts
