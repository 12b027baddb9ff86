// Generic page expansion for sm_100a: one CTA per slotted page at a time
// (persistent grid, dynamic page queue), shared by BFS, SSSP, PageRank, WCC.
//
// Paper: K_SP / K_LP (Alg 2-5) assign one warp per vertex of an
// SP (VWC) and one thread per ADJLIST entry of an LP.  B200 design
// (DESIGN.md "Kernels"): a CTA takes a whole page; an SP is processed in tiles
// of kTile consecutive slots: the tile's selected vertices (frontier test, or
// all for PageRank-like sweeps) are compacted with __ballot_sync/__popc, their
// degrees prefix-summed, and the tile's edges are then expanded edge-parallel
// (4 consecutive edges per thread, one binary search per 4 edges), so a
// degree-13 K vertex and a run of degree-1 vertices are balanced alike.  An LP
// is swept by the whole CTA; a huge vertex spans several LPs and so several
// CTAs (high-degree split).
#pragma once

#include <cstdint>
#include <type_traits>

#include "memops.cuh"
#include "runtime.h"

namespace gts {

constexpr int kThreads = 512;
constexpr int kTile = 512;
constexpr int kEdgesPerThread = 4;   // must be 4: dense tiles hand one 16-byte group per call
constexpr int kDenseUnroll = 2;      // 16-byte loads in flight per thread in dense tiles
constexpr int kWarps = kThreads / 32;

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
// same, with the encoding fixed at compile time (kVid32: entries are VIDs)
template <bool kVid32>
__device__ __forceinline__ uint32_t decode_entry_t(const PageSet& ps, uint32_t e) {
    return kVid32 ? e : __ldg(ps.rvt_start + (e >> 16)) + (e & 0xFFFFu);
}

__device__ __forceinline__ bool test_bit(const uint32_t* bm, uint32_t v) {
    return (__ldg(bm + (v >> 5)) >> (v & 31)) & 1u;
}

constexpr uint32_t kMaxTileWords = 8;   // tile mask words: up to 256 tiles (131,072 slots) per page
constexpr uint32_t kListWords = 128;    // sparse pages: frontier bitmap words compacted per pass

struct TileSmem {
    uint32_t soff[kTile + 1];  // word index of every record of the tile (all slots); soff[nv] = end
    uint8_t sel[kTile + 8];    // dense mode: vertex t of the tile is selected (4-byte aligned; +8:
                               // dense_tile_ww reads 8-byte windows up to sel[nv + 3])
    uint32_t paytile[kTile];   // dense mode: payload of vertex t of the tile
    uint32_t tmask[kMaxTileWords];   // tiles of the current page holding a frontier vertex
    uint32_t tplain[kMaxTileWords];  // tiles of the current page taken by the plain walk
    uint32_t off[kTile];       // word index of the first ADJLIST entry of item j
    uint32_t deg[kTile];
    uint32_t src[kTile];       // VID of item j
    uint32_t payload[kTile];
    uint32_t pre[kTile + 1];   // exclusive prefix of deg over items
    uint32_t wsum[kWarps];
    uint32_t wcnt[kWarps];
    uint32_t item;
    uint32_t pcount;                 // frontier vertices of the current page
    uint32_t list[kListWords * 32];  // sparse pages: compacted frontier vertices (slot indices)
};

// Tile scan: frontier compaction by __ballot_sync/__popc (position of each
// selected vertex among the tile's selected vertices) fused with the exclusive
// prefix sum of the selected vertices' degrees.  Two __syncthreads.
__device__ __forceinline__ void tile_scan(bool sel, uint32_t deg, uint32_t& pos, uint32_t& nf,
                                          uint32_t& deg_excl, uint32_t& deg_total, TileSmem& sm) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const uint32_t mask = __ballot_sync(0xFFFFFFFFu, sel);
    const uint32_t rank_in_warp = __popc(mask & ((1u << lane) - 1u));
    uint32_t x = deg;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        uint32_t y = __shfl_up_sync(0xFFFFFFFFu, x, o);
        if (lane >= o) x += y;
    }
    if (lane == 31) {
        sm.wsum[warp] = x;
        sm.wcnt[warp] = __popc(mask);
    }
    __syncthreads();
    if (warp == 0) {
        uint32_t s = lane < kWarps ? sm.wsum[lane] : 0u;
        uint32_t c = lane < kWarps ? sm.wcnt[lane] : 0u;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            uint32_t y = __shfl_up_sync(0xFFFFFFFFu, s, o);
            uint32_t z = __shfl_up_sync(0xFFFFFFFFu, c, o);
            if (lane >= o) { s += y; c += z; }
        }
        if (lane < kWarps) { sm.wsum[lane] = s; sm.wcnt[lane] = c; }   // inclusive warp prefixes
    }
    __syncthreads();
    deg_excl = (warp > 0 ? sm.wsum[warp - 1] : 0u) + x - deg;
    deg_total = sm.wsum[kWarps - 1];
    pos = (warp > 0 ? sm.wcnt[warp - 1] : 0u) + rank_in_warp;
    nf = sm.wcnt[kWarps - 1];
}

// ---- warp-window walk helpers ----
// A 128-word window of a tile's record region is one 16-byte load per lane;
// the owner of word i is j0 + #(record starts at or before i).
struct WinMask {
    uint32_t m[4];
};

// record starts in [base, base + 128) among off[j0 + 1 .. nv)
__device__ __forceinline__ WinMask win_mask(const uint32_t* off, int j0, uint32_t nv, uint32_t base, int& nstarts) {
    const int lane = threadIdx.x & 31;
    WinMask wm{{0u, 0u, 0u, 0u}};
    nstarts = 0;
    for (int r = j0 + 1;; r += 32) {
        const int j = r + lane;
        const uint32_t o = (uint32_t)j < nv ? off[j] : 0xFFFFFFFFu;
        const bool in = o - base < 128u && o >= base;
        const uint32_t p = o - base;
        const uint32_t bit = in ? 1u << (p & 31) : 0u;
        wm.m[0] |= __reduce_or_sync(0xFFFFFFFFu, (in && (p >> 5) == 0) ? bit : 0u);
        wm.m[1] |= __reduce_or_sync(0xFFFFFFFFu, (in && (p >> 5) == 1) ? bit : 0u);
        wm.m[2] |= __reduce_or_sync(0xFFFFFFFFu, (in && (p >> 5) == 2) ? bit : 0u);
        wm.m[3] |= __reduce_or_sync(0xFFFFFFFFu, (in && (p >> 5) == 3) ? bit : 0u);
        const uint32_t b = __ballot_sync(0xFFFFFFFFu, in);
        nstarts += __popc(b);
        if (b != 0xFFFFFFFFu) break;        // offsets ascend: a gap means no later start in the window
    }
    return wm;
}

// Op interface:
//   static constexpr bool kReadWeights;  -- the op needs edge weights
//   static constexpr bool kWeighted;     -- the pages carry weights (record = sz, 0, (adj, w)[sz])
//   const uint32_t* frontier()                           -- bitmap behind select(), or nullptr (all)
//   bool select(uint32_t vid)                            -- SP vertex expanded?
//   uint32_t payload(uint32_t vid, uint32_t deg)         -- per selected vertex
//   bool select_lp(uint32_t vid, uint32_t total_deg, uint32_t chunk_len, uint32_t& payload)
//   void edges(const uint32_t dst[E], const uint32_t w[E], const uint32_t pl[E], const uint32_t src[E],
//              const bool valid[E])                      -- E = kEdgesPerThread edges, loads already issued
//   void end_page()
// Edges reach the op in groups of kEdgesPerThread whose adjacency words were
// loaded back to back, so each thread has that many independent loads in
// flight, and the op can issue its own per-edge loads (visited bits, dist,
// labels) as a batch before acting on them.
// Dense-tile threshold: a tile streams its whole record region when its selected
// edges are at least kDense8 / 8 of the region's words (an op may set kDense8;
// default 4 = half).  BFS uses 6: RMAT-27 BFS kernels 7.15-7.19 ms against 7.32
// (4), 7.62 (3), 7.69 (2), 7.21 (7), 7.42 (8), 7.44 (never dense).
template <class Op, class = void>
struct dense8_of : std::integral_constant<uint32_t, 4u> {};
template <class Op>
struct dense8_of<Op, std::void_t<decltype(Op::kDense8)>> : std::integral_constant<uint32_t, Op::kDense8> {};
template <class Op>
__device__ __forceinline__ constexpr uint32_t dense_eighths() { return dense8_of<Op>::value; }

// An op with kSparseSelect = true also filters the frontier vertices of sparse pages
// through select() (default: the frontier bit alone selects them there).
template <class Op, class = void>
struct sparse_select_of : std::false_type {};
template <class Op>
struct sparse_select_of<Op, std::void_t<decltype(Op::kSparseSelect)>> : std::integral_constant<bool, Op::kSparseSelect> {};

// An op with kFastDense = true may take the plain dense walk below: a tile whose
// vertices with edges all satisfy op.done(v) (expanding any of their edges changes
// nothing the level computes) is streamed without owners or selection, and only words
// >= op.fast_floor() reach op.edges, as edges of the vertex op.plain_src() (payload
// and source alike).  An unweighted record's header is its entry count,
// so when every record of the tile has fewer entries than the floor the headers are
// filtered out with the rest and no record-start mask is needed either.
// Members such an op provides: uint32_t fast_floor() (0 = no plain walk this launch),
// bool done(v), uint32_t plain_src(), void plain_edges(selected edges of a planned run),
// uint32_t plain8 (qualifying share of selected edges, in eighths of the tile's words)
// and uint32_t plan_floor (whole-page plans from this floor up, see plan_plain_tiles).
template <class Op, class = void>
struct fast_dense_of : std::false_type {};
template <class Op>
struct fast_dense_of<Op, std::void_t<decltype(Op::kFastDense)>> : std::integral_constant<bool, Op::kFastDense> {};

constexpr int kFastUnroll = 4;       // 16-byte loads in flight per lane in the plain dense walk

// Plain dense walk (kFastDense ops, unweighted VID32 pages): window i of the tile's record
// region goes to warp i mod kWarps, one 16-byte load per lane.
template <class Op>
__device__ __forceinline__ void dense_tile_plain(Op& op, const uint4* q4, uint32_t W0, uint32_t W1, uint32_t floor,
                                                 uint64_t pol) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const uint32_t wbase = W0 & ~3u;
    const uint32_t nwin = (W1 - wbase + 127) >> 7;
    for (uint32_t wi = warp; wi < nwin; wi += kWarps * kFastUnroll) {
        uint4 vv[kFastUnroll];
#pragma unroll
        for (int u = 0; u < kFastUnroll; ++u) {
            const uint32_t q = ((wbase + ((wi + u * kWarps) << 7)) >> 2) + lane;
            vv[u] = make_uint4(0u, 0u, 0u, 0u);
            if (wi + u * kWarps < nwin && 4 * q < W1) vv[u] = ld_stream_v4(q4 + q, pol);
        }
#pragma unroll
        for (int u = 0; u < kFastUnroll; ++u) {
            const uint32_t q = ((wbase + ((wi + u * kWarps) << 7)) >> 2) + lane;
            const uint32_t ps0 = op.plain_src();
            uint32_t dst[kEdgesPerThread], wt[kEdgesPerThread] = {0u, 0u, 0u, 0u}, pl[kEdgesPerThread] = {ps0, ps0, ps0, ps0},
                     src[kEdgesPerThread] = {ps0, ps0, ps0, ps0};
            bool valid[kEdgesPerThread];
            bool any = false;
#pragma unroll
            for (int k = 0; k < 4; ++k) {
                const uint32_t w = 4 * q + k;
                dst[k] = word_of(vv[u], k);
                valid[k] = dst[k] >= floor && w >= W0 && w < W1;
                any |= valid[k];
            }
            if (any) op.edges(dst, wt, pl, src, valid);
        }
    }
}

// Edge-parallel expansion of nf compacted items (sm.off/deg/src/payload/pre):
// 4 consecutive edges per thread, one binary search per 4 edges.
template <class Op>
__device__ __forceinline__ void gather_items(const PageSet& ps, Op& op, TileSmem& sm, const uint32_t* words,
                                             uint32_t nf, uint32_t total, uint64_t pol) {
    const int tid = threadIdx.x;
    for (uint32_t e0 = (uint32_t)tid * kEdgesPerThread; e0 < total; e0 += kThreads * kEdgesPerThread) {
        uint32_t lo = 0, hi = nf;              // pre[lo] <= e0 < pre[hi]
        while (hi - lo > 1) {
            uint32_t mid = (lo + hi) >> 1;
            if (sm.pre[mid] <= e0) lo = mid; else hi = mid;
        }
        uint32_t j = lo, nxt = sm.pre[lo + 1];
        uint32_t dst[kEdgesPerThread], w[kEdgesPerThread], pl[kEdgesPerThread], src[kEdgesPerThread];
        bool valid[kEdgesPerThread];
#pragma unroll
        for (int q = 0; q < kEdgesPerThread; ++q) {
            const uint32_t e = e0 + q;
            valid[q] = e < total;
            if (valid[q]) {
                while (e >= nxt) nxt = sm.pre[++j + 1];
            }
            const uint32_t local = e - sm.pre[j];
            const uint32_t* adj = words + sm.off[j];
            if (Op::kWeighted) {                // (neighbour, weight): one 8-byte load
                const uint2 pr = valid[q] ? ld_stream_l1_v2(adj + 2 * local, pol) : make_uint2(0u, 0u);
                dst[q] = pr.x;
                w[q] = pr.y;
            } else {
                dst[q] = valid[q] ? ld_stream_l1_u32(adj + local, pol) : 0u;
                w[q] = 0u;
            }
            pl[q] = sm.payload[j];
            src[q] = sm.src[j];
        }
#pragma unroll
        for (int q = 0; q < kEdgesPerThread; ++q) dst[q] = decode_entry(ps, dst[q]);
        op.edges(dst, w, pl, src, valid);
    }
}

// Sparse page (frontier-driven ops, < 1/4 of the page's vertices selected):
// compact the page's frontier vertices from the bitmap in passes of
// kListWords words, then expand them in batches of kTile with gather_items.
template <class Op>
__device__ void expand_sparse_page(const PageSet& ps, Op& op, TileSmem& sm, const uint8_t* data,
                                   const uint8_t* end, uint32_t start, uint32_t nslots, const uint32_t* fbm,
                                   uint64_t pol) {
    const int tid = threadIdx.x;
    const uint32_t* words = reinterpret_cast<const uint32_t*>(data);
    const uint32_t w0 = start >> 5, w1 = (start + nslots - 1) >> 5;
    for (uint32_t wb = w0; wb <= w1; wb += kListWords) {
        const uint32_t w = wb + tid;
        uint32_t bits = 0;
        if ((uint32_t)tid < kListWords && w <= w1) {
            bits = __ldg(fbm + w);
            if (w == w0) bits &= 0xFFFFFFFFu << (start & 31);
            if (w == w1 && ((start + nslots) & 31)) bits &= 0xFFFFFFFFu >> (32 - ((start + nslots) & 31));
        }
        uint32_t pos, nw, excl, tot;
        tile_scan(bits != 0, __popc(bits), pos, nw, excl, tot, sm);
        uint32_t k = excl;
        while (bits) {
            const uint32_t b = __ffs(bits) - 1;
            sm.list[k++] = w * 32 + b - start;
            bits &= bits - 1;
        }
        __syncthreads();
        for (uint32_t b0 = 0; b0 < tot; b0 += kTile) {
            const uint32_t kk = b0 + tid;
            bool sel = kk < tot;
            uint32_t j = sel ? sm.list[kk] : 0u, off = 0, deg = 0;
            if constexpr (sparse_select_of<Op>::value) sel = sel && op.select(start + j);
            if (sel) {
                const uint8_t* slot = end - kSpFooter - kSlotBytes * (uint64_t)(j + 1);
                off = ld_stream_u32(slot + 4, pol);
                deg = ld_stream_u32(data + off, pol) ;
            }
            const uint32_t v = start + j;
            const uint32_t pay = sel ? op.payload(v, deg) : 0u;
            const bool item = sel && deg > 0;            // items with edges only
            uint32_t p2, nf, ex2, total;
            tile_scan(item, item ? deg : 0u, p2, nf, ex2, total, sm);
            if (item) {
                sm.off[p2] = off / 4 + rec_hdr_words(Op::kWeighted);
                sm.deg[p2] = deg;
                sm.src[p2] = v;
                sm.payload[p2] = pay;
                sm.pre[p2] = ex2;
            }
            if (tid == 0) sm.pre[nf] = total;
            __syncthreads();
            gather_items(ps, op, sm, words, nf, total, pol);
            // no barrier here: the gather reads only the item arrays, and the next batch
            // rewrites them only after its tile_scan barriers, which every thread reaches
            // after finishing this gather
        }
    }
}

// ---- the paper's micro-level techniques (App E / Fig 14) ----
// Kept beside the tile engine for the Fig 14 comparison (GTS_MICRO_* run flags):
//   edge-centric   = VWC with W_SZ = 32 (Alg 2 l.9-11, R8): a warp per vertex of
//                    the SP, its lanes strided over the ADJLIST;
//   vertex-centric = a thread per vertex and its entire ADJLIST;
//   hybrid         = per page by density: vertex-centric if the page's edges per
//                    vertex are below ps.hybrid_deg, else edge-centric (R24).
// Every vertex of the page is tested (Alg 2 l.12 tests LV of each vertex).
enum { kMicroTile = 0, kMicroEdge = 1, kMicroVertex = 2, kMicroHybrid = 3 };

template <class Op>
__device__ __forceinline__ void micro_edges(const PageSet& ps, Op& op, const uint32_t* adj, uint32_t deg,
                                            uint32_t k0, uint32_t stride, uint32_t pay, uint32_t v, uint64_t pol) {
    uint32_t dst[kEdgesPerThread], w[kEdgesPerThread], pl[kEdgesPerThread], src[kEdgesPerThread];
    bool valid[kEdgesPerThread];
#pragma unroll
    for (int q = 0; q < kEdgesPerThread; ++q) {
        const uint32_t k = k0 + q * stride;
        valid[q] = k < deg;
        if (Op::kWeighted) {
            const uint2 pr = valid[q] ? ld_stream_v2(adj + 2 * k, pol) : make_uint2(0u, 0u);
            dst[q] = pr.x;
            w[q] = pr.y;
        } else {
            dst[q] = valid[q] ? ld_stream_u32(adj + k, pol) : 0u;
            w[q] = 0u;
        }
        pl[q] = pay;
        src[q] = v;
    }
#pragma unroll
    for (int q = 0; q < kEdgesPerThread; ++q) dst[q] = decode_entry(ps, dst[q]);
    op.edges(dst, w, pl, src, valid);
}

template <class Op, int kMicro>
__device__ void expand_sp_micro(const PageSet& ps, Op& op, const uint8_t* data, const uint8_t* end,
                                uint32_t nslots, uint64_t pol) {
    const uint32_t* words = reinterpret_cast<const uint32_t*>(data);
    const uint32_t start = ld32(end - kSpFooter - kSlotBytes);
    constexpr uint32_t wsh = Op::kWeighted ? 1 : 0, hdr = rec_hdr_words(Op::kWeighted);
    bool vertex = kMicro == kMicroVertex;
    if (kMicro == kMicroHybrid) {              // page density from its last record's end
        const uint32_t lo = ld32(end - kSpFooter - kSlotBytes * (uint64_t)nslots + 4);
        const uint32_t used = lo / 4 + hdr + (ld32(data + lo) << wsh);     // record words
        const uint32_t nedges = (used - hdr * nslots) >> wsh;
        vertex = nedges < ps.hybrid_deg * nslots;
    }
    if (vertex) {
        for (uint32_t u = threadIdx.x; u < nslots; u += kThreads) {
            const uint32_t v = start + u;
            if (!op.select(v)) continue;
            const uint32_t off = ld_stream_u32(end - kSpFooter - kSlotBytes * (uint64_t)(u + 1) + 4, pol);
            const uint32_t deg = ld_stream_u32(data + off, pol);
            const uint32_t pay = op.payload(v, deg);
            const uint32_t* adj = words + off / 4 + hdr;
            for (uint32_t k0 = 0; k0 < deg; k0 += kEdgesPerThread) micro_edges(ps, op, adj, deg, k0, 1, pay, v, pol);
        }
    } else {
        const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
        for (uint32_t u = warp; u < nslots; u += kWarps) {       // warp-uniform loop
            const uint32_t v = start + u;
            if (!op.select(v)) continue;
            const uint32_t off = ld_stream_u32(end - kSpFooter - kSlotBytes * (uint64_t)(u + 1) + 4, pol);
            const uint32_t deg = ld_stream_u32(data + off, pol);
            uint32_t pay = lane == 0 ? op.payload(v, deg) : 0u;
            pay = __shfl_sync(0xFFFFFFFFu, pay, 0);
            const uint32_t* adj = words + off / 4 + hdr;
            for (uint32_t k0 = lane; k0 < deg; k0 += 32 * kEdgesPerThread) micro_edges(ps, op, adj, deg, k0, 32, pay, v, pol);
        }
    }
}

// Dense tile by warp windows (sm.soff / sm.sel / sm.paytile of the tile are
// published).  Same per-edge contract as the tile walk: op.edges gets the 4
// words of one 16-byte load per call.
template <class Op, bool kVid32>
__device__ __forceinline__ void dense_tile_ww(const PageSet& ps, Op& op, TileSmem& sm, const uint4* q4,
                                              const uint32_t* words, uint32_t v0, uint32_t nv, uint32_t W0,
                                              uint32_t W1, uint64_t pol) {
    constexpr uint32_t wsh = Op::kWeighted ? 1 : 0;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const uint32_t wbase = W0 & ~3u;
    const uint32_t nwin = (W1 - wbase + 127) >> 7;
    const uint32_t per = (nwin + kWarps - 1) / kWarps;
    const uint32_t wa = min(nwin, warp * per), wb = min(nwin, wa + per);
    if (wa >= wb) return;
    const uint32_t base0 = wbase + (wa << 7);
    int lo = -1, hi = (int)nv;                      // soff[lo] < base0 <= soff[hi]
    while (hi - lo > 1) {
        const int mid = (lo + hi) >> 1;
        if (sm.soff[mid] < base0) lo = mid; else hi = mid;
    }
    int j0 = lo;
    for (uint32_t wi = wa; wi < wb; wi += kDenseUnroll) {
        uint4 vv[kDenseUnroll];
#pragma unroll
        for (int u = 0; u < kDenseUnroll; ++u) {
            const uint32_t q = ((wbase + ((wi + u) << 7)) >> 2) + lane;
            vv[u] = make_uint4(0u, 0u, 0u, 0u);
            if (wi + u < wb && 4 * q < W1) vv[u] = ld_stream_v4(q4 + q, pol);
        }
#pragma unroll
        for (int u = 0; u < kDenseUnroll; ++u) {
            if (wi + u >= wb) break;
            const uint32_t bw = wbase + ((wi + u) << 7);
            const uint32_t q = (bw >> 2) + lane;
            int ns;
            const WinMask wm = win_mask(sm.soff, j0, nv, bw, ns);
            const uint32_t mw = lane >> 3;
            uint32_t before = 0;
#pragma unroll
            for (int k = 0; k < 4; ++k) before += (uint32_t)k < mw ? __popc(wm.m[k]) : 0u;
            const uint32_t mword = mw == 0 ? wm.m[0] : mw == 1 ? wm.m[1] : mw == 2 ? wm.m[2] : wm.m[3];
            uint32_t dst[kEdgesPerThread], wt[kEdgesPerThread], pl[kEdgesPerThread], src[kEdgesPerThread];
            bool valid[kEdgesPerThread];
            if (!Op::kWeighted) {
                // Unweighted records: every non-start word of a record is an entry.  The
                // lane's 4 words have owners jb + c (c = record starts up to the word), so
                // sel[jb .. jb+4] comes from one 8-byte window of sm.sel (two aligned LDS)
                // instead of a dependent LDS.U8 per word.  selw = sm.sel - 4 bytes (jb >= -1).
                const uint32_t bpos0 = (4 * lane) & 31;
                const uint32_t nb = (mword >> bpos0) & 0xFu;           // record starts among my words
                const int jb = j0 + (int)(before + __popc(mword & ((1u << bpos0) - 1u)));
                const uint32_t t = (uint32_t)(jb + 4);
                const uint32_t* selw = reinterpret_cast<const uint32_t*>(sm.sel) - 1;
                const unsigned long long sw =
                    ((unsigned long long)selw[(t >> 2) + 1] << 32 | selw[t >> 2]) >> (8 * (t & 3));
                uint32_t c = 0;
#pragma unroll
                for (int k = 0; k < 4; ++k) {
                    const uint32_t w = 4 * q + k;
                    const uint32_t st = (nb >> k) & 1u;
                    c += st;
                    valid[k] = !st && w >= W0 && w < W1 && ((sw >> (8 * c)) & 0xFFu);
                    wt[k] = 0u;
                    dst[k] = decode_entry_t<kVid32>(ps, word_of(vv[u], k));
                    const int j = jb + (int)c;
                    pl[k] = valid[k] ? sm.paytile[j] : 0u;
                    src[k] = v0 + (uint32_t)j;
                }
                op.edges(dst, wt, pl, src, valid);
                j0 += ns;
                continue;
            }
            // Weighted records (sz, 0, (adj, w) pairs), 8-byte aligned: a word is an entry iff
            // it lies past its owner's 2-word header at an even distance from the record start,
            // and its weight is the next word of the same 16-byte group (k = 0 or 2 only).
            const uint32_t bpos0 = (4 * lane) & 31;
            const uint32_t nb = (mword >> bpos0) & 0xFu;
            const int jb = j0 + (int)(before + __popc(mword & ((1u << bpos0) - 1u)));
            uint32_t c = 0;
#pragma unroll
            for (int k = 0; k < 4; ++k) {
                const uint32_t w = 4 * q + k;
                const uint32_t st = (nb >> k) & 1u;
                c += st;
                const int j = jb + (int)c;
                // (record starts are even words, so w - start is even iff k is even)
                const bool ok = !st && !(k & 1) && w >= W0 && w < W1 && w - sm.soff[j] >= 2 && sm.sel[j];
                wt[k] = ok ? word_of(vv[u], k + 1) : 0u;
                valid[k] = ok;
                dst[k] = decode_entry_t<kVid32>(ps, word_of(vv[u], k));
                pl[k] = ok ? sm.paytile[j] : 0u;
                src[k] = v0 + (uint32_t)j;
            }
            op.edges(dst, wt, pl, src, valid);
            j0 += ns;
        }
    }
}

// Plain-walk plan of one SP (kFastDense ops, levels with a probe floor): one pass over the
// page's slots marks the tiles that qualify -- every vertex with edges satisfies op.done(v)
// and has fewer entries than the floor, and the selected edges are >= op.plain8 / 8 of the
// tile's record words -- in sm.tplain, and leaves each tile's first record word in
// tstart[t] (tstart[ntiles] = end of the page's records) and its selected edges in tsum[t]
// (both in sm.list, which only sparse pages use).  Runs of consecutive plain tiles are then
// streamed as one range: no per-tile setup and one barrier per run.
template <class Op>
__device__ __forceinline__ void plan_plain_tiles(Op& op, TileSmem& sm, const uint8_t* data, const uint8_t* end,
                                                 uint32_t start, uint32_t nslots, uint32_t ntiles,
                                                 const uint32_t* fbm, uint32_t floor, uint64_t pol) {
    const int tid = threadIdx.x, lane = tid & 31;
    uint32_t* tsum = sm.list;
    uint32_t* tstart = sm.list + 32 * kMaxTileWords;
    uint32_t* tbad = sm.list + 64 * kMaxTileWords + 1;
    for (uint32_t k = tid; k < ntiles; k += kThreads) tsum[k] = 0u;
    for (uint32_t k = tid; k < kMaxTileWords; k += kThreads) tbad[k] = 0u;
    __syncthreads();
    for (uint32_t j0 = 0; j0 < nslots; j0 += kThreads) {     // uniform trip count
        const uint32_t j = j0 + tid;
        const bool in = j < nslots;
        uint32_t o = 0;
        if (in) o = ld_stream_u32(end - kSpFooter - kSlotBytes * (uint64_t)(j + 1) + 4, pol) >> 2;
        uint32_t on = __shfl_down_sync(0xFFFFFFFFu, o, 1);
        if (in && (lane == 31 || j + 1 == nslots)) {
            if (j + 1 < nslots) on = ld_stream_u32(end - kSpFooter - kSlotBytes * (uint64_t)(j + 2) + 4, pol) >> 2;
            else on = o + 1 + ld32(data + 4ull * o);             // unweighted record: header = entry count
        }
        const uint32_t deg = in ? on - o - 1 : 0u;
        const uint32_t v = start + j, t = j0 / kTile;            // a warp's vertices share one tile
        if (in && (j & (kTile - 1)) == 0) tstart[t] = o;
        if (in && j + 1 == nslots) tstart[ntiles] = on;
        const bool sel = in && deg > 0 && (!fbm || test_bit(fbm, v));
        uint32_t se = sel ? deg : 0u;
#pragma unroll
        for (int d = 16; d > 0; d >>= 1) se += __shfl_down_sync(0xFFFFFFFFu, se, d);
        if (lane == 0 && se) atomicAdd(&tsum[t], se);
        const bool bad = in && deg > 0 && !(deg < floor && op.done(v));
        if (__any_sync(0xFFFFFFFFu, bad) && lane == 0) atomicOr(&tbad[t >> 5], 1u << (t & 31));
    }
    __syncthreads();
    for (uint32_t k = tid; k < kMaxTileWords; k += kThreads) {
        uint32_t m = 0;
        for (uint32_t b = 0; b < 32; ++b) {
            const uint32_t t = 32 * k + b;
            if (t < ntiles && !((tbad[k] >> b) & 1u) && 8ull * tsum[t] >= (uint64_t)op.plain8 * (tstart[t + 1] - tstart[t]) &&
                tsum[t] > 0)
                m |= 1u << b;
        }
        sm.tplain[k] = m;
    }
    __syncthreads();
}

template <class Op, int kMicro = kMicroTile>
__device__ void expand_pages(const PageSet& ps, Op& op, TileSmem& sm, uint32_t* work_ctr) {
    const uint32_t npages = ps.d_count ? *(volatile const uint32_t*)ps.d_count : ps.count;
    // work items per page: ps.split, or 0 = automatic: slice LPs when the set has fewer
    // than half as many pages as the grid has CTAs (same value in every CTA)
    const uint32_t S = ps.split ? ps.split
                                : (npages > 0 && 2 * npages < gridDim.x ? min(64u, gridDim.x / npages) : 1u);
    const uint32_t count = npages * S;
    const int tid = threadIdx.x;
    const uint64_t pol = policy_evict_first();
    uint32_t ffloor = 0;                 // plain dense walk: probe floor (0 = not this launch)
    if constexpr (fast_dense_of<Op>::value) {
        ffloor = op.fast_floor();
        if (ps.entry_encoding != GTS_ENTRY_VID32) ffloor = 0;
    }
    for (;;) {
        if (tid == 0) sm.item = atomicAdd(work_ctr, 1u);
        __syncthreads();
        const uint32_t item = sm.item;
        __syncthreads();
        if (item >= count) break;
        const uint32_t i = S == 1 ? item : item / S, sub = S == 1 ? 0u : item % S;
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
            // slice `sub` of S of the chunk (high-degree split across CTAs)
            const uint32_t klo = (uint32_t)((uint64_t)len * sub / S), khi = (uint32_t)((uint64_t)len * (sub + 1) / S);
            uint32_t payload = 0;
            if (khi > klo && op.select_lp(vid, total, khi - klo, payload)) {
                const uint32_t* adj = words + rec_hdr_words(Op::kWeighted);
                for (uint32_t k0 = klo + tid; k0 < khi; k0 += kThreads * kEdgesPerThread) {
                    uint32_t dst[kEdgesPerThread], w[kEdgesPerThread], pl[kEdgesPerThread], src[kEdgesPerThread];
                    bool valid[kEdgesPerThread];
#pragma unroll
                    for (int q = 0; q < kEdgesPerThread; ++q) {
                        const uint32_t k = k0 + q * kThreads;
                        valid[q] = k < khi;
                        if (Op::kWeighted) {
                            const uint2 pr = valid[q] ? ld_stream_v2(adj + 2 * k, pol) : make_uint2(0u, 0u);
                            dst[q] = pr.x;
                            w[q] = pr.y;
                        } else {
                            dst[q] = valid[q] ? ld_stream_u32(adj + k, pol) : 0u;
                            w[q] = 0u;
                        }
                        pl[q] = payload;
                        src[q] = vid;
                    }
#pragma unroll
                    for (int q = 0; q < kEdgesPerThread; ++q) dst[q] = decode_entry(ps, dst[q]);
                    op.edges(dst, w, pl, src, valid);
                }
            }
        } else if (sub != 0) {
            continue;                           // an SP is one work item (slice 0)
        } else if (kMicro != kMicroTile) {
            expand_sp_micro<Op, kMicro>(ps, op, data, end, nslots, pol);
        } else {
            const uint32_t start = ld32(end - kSpFooter - kSlotBytes);
            const uint4* q4 = reinterpret_cast<const uint4*>(data);
            const uint32_t ntiles = (nslots + kTile - 1) / kTile;
            // Frontier-driven ops: one pass over the page's frontier-bitmap words marks
            // the tiles that hold a selected vertex, so inactive tiles cost nothing.
            const uint32_t* fbm = ntiles <= 32 * kMaxTileWords ? op.frontier() : nullptr;
            if (fbm) {
                for (uint32_t k = tid; k < kMaxTileWords; k += kThreads) sm.tmask[k] = 0u;
                if (tid == 0) sm.pcount = 0;
                __syncthreads();
                uint32_t cnt = 0;
                const uint32_t w0 = start >> 5, w1 = (start + nslots - 1) >> 5;
                for (uint32_t w = w0 + tid; w <= w1; w += kThreads) {
                    uint32_t bits = __ldg(fbm + w);
                    if (w == w0) bits &= 0xFFFFFFFFu << (start & 31);
                    if (w == w1 && ((start + nslots) & 31)) bits &= 0xFFFFFFFFu >> (32 - ((start + nslots) & 31));
                    cnt += __popc(bits);
                    if (bits) {
                        const uint32_t a = w * 32 + (__ffs(bits) - 1) - start;
                        const uint32_t b = w * 32 + (31 - __clz(bits)) - start;
                        for (uint32_t t = a / kTile; t <= b / kTile; ++t) atomicOr(&sm.tmask[t >> 5], 1u << (t & 31));
                    }
                }
                if (cnt) atomicAdd(&sm.pcount, cnt);
                __syncthreads();
                if (4 * sm.pcount < nslots) {          // uniform: sparse page -> compacted batches
                    expand_sparse_page(ps, op, sm, data, end, start, nslots, fbm, pol);
                    op.end_page();
                    continue;
                }
            }
            bool plain = false;                   // this page has a plain-walk plan (sm.tplain)
            if constexpr (fast_dense_of<Op>::value) {
                if (ffloor >= op.plan_floor && ntiles <= 32 * kMaxTileWords) {
                    plan_plain_tiles(op, sm, data, end, start, nslots, ntiles, fbm, ffloor, pol);
                    plain = true;
                }
            }
            auto is_plain = [&](uint32_t t) { return plain && ((sm.tplain[t >> 5] >> (t & 31)) & 1u); };
            auto active = [&](uint32_t t) { return !fbm || ((sm.tmask[t >> 5] >> (t & 31)) & 1u); };
            auto next_active = [&](uint32_t t) {
                while (t < ntiles && !active(t)) ++t;     // uniform: tiles without a frontier vertex cost nothing
                return t;
            };
            // (Staging the next active tile's slot array into shared memory with a 1D TMA copy
            // -- cp.async.bulk + mbarrier, double-buffered, one elected thread -- measured
            // slower on RMAT-27: BFS 7.41 vs 7.36 ms, WCC 12.84 vs 12.64 ms; the slot loads are
            // not what these kernels wait on.)
            for (uint32_t ti = next_active(0); ti < ntiles; ti = next_active(ti + 1)) {
                if constexpr (fast_dense_of<Op>::value) {
                    if (is_plain(ti)) {                   // uniform: a run of plain tiles, one range
                        uint32_t tj = ti + 1, se = sm.list[ti];
                        while (tj < ntiles && is_plain(tj)) se += sm.list[tj++];
                        const uint32_t* tstart = sm.list + 32 * kMaxTileWords;
                        dense_tile_plain(op, q4, tstart[ti], tstart[tj], ffloor, pol);
                        if (tid == 0) op.plain_edges(se);
                        __syncthreads();
                        ti = tj - 1;
                        continue;
                    }
                }
                const uint32_t t0 = ti * kTile;
                const uint32_t nv = min((uint32_t)kTile, nslots - t0);
                const uint32_t v = start + t0 + tid;
                const bool sel = (uint32_t)tid < nv && op.select(v);
                // record offsets of the whole tile; the degree of a record is the distance to
                // the next record (the last one reads its header)
                if ((uint32_t)tid < nv) {                // coalesced slot reads
                    const uint8_t* slot = end - kSpFooter - kSlotBytes * (uint64_t)(t0 + tid + 1);
                    const uint32_t o = ld_stream_u32(slot + 4, pol);
                    sm.soff[tid] = o >> 2;
                    if ((uint32_t)tid == nv - 1) {
                        if (t0 + nv < nslots) sm.soff[nv] = ld_stream_u32(slot - kSlotBytes + 4, pol) >> 2;
                        else sm.soff[nv] = (o >> 2) + rec_hdr_words(Op::kWeighted) + (ld32(data + o) << (Op::kWeighted ? 1 : 0));
                    }
                }
                if (!__syncthreads_or(sel)) continue;   // (also publishes soff)
                uint32_t deg = 0;
                if ((uint32_t)tid < nv)
                    deg = (sm.soff[tid + 1] - sm.soff[tid] - rec_hdr_words(Op::kWeighted)) >> (Op::kWeighted ? 1 : 0);
                const uint32_t pay = sel ? op.payload(v, deg) : 0u;
                if ((uint32_t)tid < nv) {               // published by tile_scan's barriers
                    sm.sel[tid] = sel ? 1 : 0;
                    sm.paytile[tid] = pay;
                }
                uint32_t pos, nf, excl, total;
                const bool item = sel && deg > 0;        // sparse tiles compact items with edges only
                tile_scan(item, item ? deg : 0u, pos, nf, excl, total, sm);
                const uint32_t W0 = sm.soff[0], W1 = sm.soff[nv];
                // dense: the selected edges are >= half of the tile's record words.  Weighted
                // records hold 2 words per edge, so there a tile is dense only when nearly
                // every vertex is selected -- measured the better choice for SSSP (RMAT-27
                // 35.7 ms vs 42.8 ms when the selected words are counted instead; with the
                // interleaved (adj, w) records 33.5 vs 35.3 ms)
                const bool dense = 8 * total >= dense_eighths<Op>() * (W1 - W0);
                if constexpr (fast_dense_of<Op>::value) {
                    // no page plan (small floor): the same test per tile, after its setup
                    if (!plain && ffloor && 8 * total >= op.plain8 * (W1 - W0) &&
                        __syncthreads_and((uint32_t)tid >= nv || deg == 0 || (deg < ffloor && op.done(v)))) {
                        dense_tile_plain(op, q4, W0, W1, ffloor, pol);
                        continue;           // (the plain walk reads no shared memory: no barrier)
                    }
                }
                if (dense) {
                    // dense tile, warp-window walk: each warp streams a contiguous run of
                    // 128-word windows; owners from record-start masks (no binary search;
                    // RMAT-27 SSSP 33.8 vs 36.2 ms, WCC 13.7 vs 14.2 ms against a binary
                    // search per 16 bytes, BFS equal)
                    if (ps.entry_encoding == GTS_ENTRY_VID32)
                        dense_tile_ww<Op, true>(ps, op, sm, q4, words, start + t0, nv, W0, W1, pol);
                    else
                        dense_tile_ww<Op, false>(ps, op, sm, q4, words, start + t0, nv, W0, W1, pol);
                    __syncthreads();
                    continue;
                }
                // sparse tile: compacted selected vertices, edge-parallel gather
                if (item) {
                    sm.off[pos] = sm.soff[tid] + rec_hdr_words(Op::kWeighted);
                    sm.deg[pos] = deg;
                    sm.src[pos] = v;
                    sm.payload[pos] = pay;
                    sm.pre[pos] = excl;
                }
                if (tid == 0) sm.pre[nf] = total;
                __syncthreads();
                gather_items(ps, op, sm, words, nf, total, pol);
                // (no trailing barrier: the next tile rewrites the item arrays only after its
                // own tile_scan barriers; its soff / sel / paytile writes are not read here)
            }
        }
        op.end_page();
    }
}

}  // namespace gts
