// PageRank over slotted pages.
//
// Paper: K_PR_SP / K_PR_LP (Alg 4/5): for every edge u->v of the
// page, atomicAdd(nextPR[v], df * prevPR[u] / ADJLIST_SZ(u)), with nextPR
// initialised to (1-df)/|V| before the kernels and copied to
// prevPR after each iteration.  prevPR is RA, nextPR is WA.
//
// B200 design:
//  * pr_scatter: persistent CTAs over pages (expand.cuh); per selected vertex
//    c_u = d * x_u / outdeg(u) (LP: divided by the TOTAL degree, R4); per edge
//    a fire-and-forget fp32 red.add into acc (WA).  Runs of equal destinations
//    inside a thread (rows are sorted) are combined first.  Destinations in the
//    graph's hot table (top in-degree vertices) are pre-aggregated per CTA in
//    shared memory and flushed with one global add per CTA: this bounds the
//    number of fp32 additions into a hub to ~#CTAs (the fp32 error gate at
//    RMAT-27+ hubs, SURVEY section 7 hard parts) and removes the most
//    contended global atomics.
//  * dangling mass D (sum of x_u over outdeg(u) = 0, R3) is reduced in fp64.
//  * pr_finish (fused damping / dangling / swap): x_v = (1-d)/n + d*D/n + acc_v,
//    acc_v = 0.  Teleport and D are applied once, after the merge, so
//    Strategy-P replicas add edge terms only (R17).
#include <cuda_runtime.h>
#include <nccl.h>

#include <algorithm>
#include <array>
#include <cstdlib>
#include <cstring>

#include "comm.h"
#include "expand.cuh"
#include "memops.cuh"
#include "route.cuh"
#include "sweep.cuh"

namespace gts {

// Hot-destination modes of the scatter:
//   kHash    : natural VID order; the builder's top-4096 in-degree vertices in a
//              bucketed two-choice hash table in shared memory
//   kDense   : degree-ordered pages; hot = internal IDs [0, kHotDense), one
//              shared-memory array per CTA
// (A third mode that spread a 4x larger hot set over the distributed shared
// memory of a 4-CTA cluster with red.shared::cluster was built and measured:
// 2.2x slower on RMAT-27 and a larger fp32 error at the hub; removed.)
//   kRoute   : Strategy-S with routed updates (SURVEY 8(e) "S-route"): dense hot set
//              as kDense; destinations in this rank's WA range [lo, hi) are added
//              locally, all others are packed into per-owner (dst, value) buffers
//              that the driver exchanges with NCCL send/recv; hot partial sums for
//              non-local hot vertices go to a dense per-rank buffer reduced onto
//              their owners.
//   kRouteHash: Strategy-S on natural-order pages: the hash hot set of kHash with the
//              owner routing of kRoute (the hubs are not the low IDs there, and without
//              per-CTA aggregation a hub's fp32 sum takes millions of sequential adds)
enum PrMode : int { kHash = 0, kDense = 1, kRoute = 2, kRouteHash = 3 };

struct RouteParams {
    float* acc_loc;                    // local WA, biased: acc_loc[v] for v in [lo, hi)
    float* hot_out;                    // [n_hot] hot partial sums of vertices outside [lo, hi)
    uint64_t lo, hi;
    int drop_remote;                   // paper-literal Strategy-S (every page on every rank): drop remote updates
    int direct;                        // GTS_ROUTE_PEER: remote updates are atomics into the owner's WA
    RouteOut ro;                       // Strategy-S: (dst, value) messages to the owners (ro.vr: the ranges)
    float* peer_acc[kMaxRanks];        // GTS_ROUTE_PEER: every owner's WA (biased, peer memory)
};

// Per-thread destination emitter: combines runs of equal destinations (rows
// are sorted), routes hot destinations to shared-memory partial sums and
// everything else to a fire-and-forget fp32 red.add into acc.
template <int kMode, uint32_t H>
struct PrEmitter {
    float* acc;
    const uint32_t* hkeys;   // kHash: shared memory keys
    float* hacc;             // shared memory partial sums
    const RouteParams* rp;   // kRoute
    uint32_t last;
    float sum;
    bool has;

    __device__ __forceinline__ void emit(uint32_t dst, float c) {
        if (kMode == kRoute) {
            if (dst < H) atomicAdd(hacc + dst, c);
            else cold(dst, c);
            return;
        }
        if (kMode == kDense) {
            if (dst < H) atomicAdd(hacc + dst, c);
            else atomicAdd(acc + dst, c);
            return;
        }
        uint32_t b = hot_h1(dst);
        uint4 k = reinterpret_cast<const uint4*>(hkeys)[b];
        int way = k.x == dst ? 0 : k.y == dst ? 1 : k.z == dst ? 2 : k.w == dst ? 3 : -1;
        if (way < 0 && k.w != kHotEmpty) {              // h1 full: the key may sit in h2
            b = hot_h2(dst);
            k = reinterpret_cast<const uint4*>(hkeys)[b];
            way = k.x == dst ? 0 : k.y == dst ? 1 : k.z == dst ? 2 : k.w == dst ? 3 : -1;
        }
        if (way >= 0) atomicAdd(hacc + b * kHotWays + way, c);
        else if (kMode == kRouteHash) cold(dst, c);
        else atomicAdd(acc + dst, c);                   // REDG.E.ADD.F32 (result unused)
    }
    // Strategy-S: a destination outside the hot set, to this rank's WA or to its owner
    __device__ __forceinline__ void cold(uint32_t dst, float c) {
        if ((uint64_t)dst >= rp->lo && (uint64_t)dst < rp->hi) atomicAdd(rp->acc_loc + dst, c);
        else if (rp->direct) atomicAdd(rp->peer_acc[route_owner(rp->ro, dst)] + dst, c);   // over NVLink
        else if (!rp->drop_remote) route_push<uint2>(rp->ro, dst, make_uint2(dst, __float_as_uint(c)));
    }
    __device__ __forceinline__ void edge(uint32_t dst, float c) {
        if (has && dst == last) {
            sum += c;
            return;
        }
        if (has) emit(last, sum);
        last = dst;
        sum = c;
        has = true;
    }
    __device__ __forceinline__ void flush() {
        if (has) emit(last, sum);
        has = false;
    }
};

constexpr int kPrUnroll = 4;            // 16-byte loads in flight per thread

template <int T>
struct PrSmem {
    uint32_t off[T + 1];                // page-relative word index of each record of the tile; off[nv] = end
    float c[T];                         // d * x_u / outdeg(u)
    uint32_t item;
};

template <int kMode, uint32_t H>
constexpr size_t pr_dyn_smem() {
    return (kMode == kHash || kMode == kRouteHash) ? kHotSlots * (sizeof(uint32_t) + sizeof(float))
                                                   : H * sizeof(float);   // kDense, kRoute
}

// dense hot-set sizes: 512-thread CTAs (2 per SM) hold kHotDense floats each;
// 1024-thread CTAs (1 per SM) hold kHotDenseBig
constexpr uint32_t kHotDenseBig = 53248;
// vertices per thread in a scatter tile (1024-thread CTAs: 2048-vertex tiles)
constexpr int kPrVpt = 2;

template <bool kVid32>
__device__ __forceinline__ uint32_t pr_decode(uint32_t e, const uint32_t* rvt) {
    return kVid32 ? e : __ldg(rvt + (e >> 16)) + (e & 0xFFFFu);
}

// K_PR_SP / K_PR_LP (Alg 4/5) for a persistent CTA of T threads.  The record
// region of a tile of T consecutive vertices is one contiguous word range
// (records are packed in VID order from offset 0), streamed with 16-byte
// evict_first loads, kPrUnroll in flight per thread; the owner of each 4-word
// group is found by a binary search over the tile's record offsets.
template <bool kWeighted, int kMode, int T, int kMinBlocks, uint32_t H, int VPT, bool kVid>
__global__ void __launch_bounds__(T, kMinBlocks)
pr_scatter_kernel(PageSet ps, const float* __restrict__ x, float* acc, const uint32_t* __restrict__ hot_keys,
                  float d, double* dang_out, uint32_t* work_ctr, uint32_t n_hot, const RouteParams rp) {
    __shared__ PrSmem<T * VPT> sm;
    extern __shared__ uint4 dyn_smem[];
    uint32_t* hkeys = reinterpret_cast<uint32_t*>(dyn_smem);
    constexpr bool kHashed = kMode == kHash || kMode == kRouteHash;
    float* hacc = kHashed ? reinterpret_cast<float*>(hkeys + kHotSlots) : reinterpret_cast<float*>(dyn_smem);
    const int tid = threadIdx.x;
    if (kHashed) {
        for (uint32_t i = tid; i < kHotSlots; i += T) {
            hkeys[i] = __ldg(hot_keys + i);
            hacc[i] = 0.f;
        }
    } else {
        for (uint32_t i = tid; i < H; i += T) hacc[i] = 0.f;
    }
    __syncthreads();
    const uint64_t pol = policy_evict_first();
    const uint32_t count = ps.count;
    constexpr uint32_t wshift = kWeighted ? 1 : 0;
    PrEmitter<kMode, H> em{acc, hkeys, hacc, &rp, 0u, 0.f, false};
    double dang = 0.0;
    for (;;) {
        if (tid == 0) sm.item = atomicAdd(work_ctr, 1u);
        __syncthreads();
        const uint32_t it = sm.item;
        __syncthreads();                     // sm.item is rewritten by thread 0 next round
        if (it >= count) break;
        uint32_t pid;
        const uint8_t* data;
        page_at(ps, it, pid, data);
        const uint8_t* end = data + ps.page_bytes;
        const uint32_t kind = ld32(end - 4);
        const uint32_t nslots = ld32(end - 8);
        const uint4* q4 = reinterpret_cast<const uint4*>(data);
        if (kind == GTS_PAGE_LP) {
            const uint32_t vid = ld32(end - kLpFooter - kSlotBytes);
            const uint32_t total = ld32(end - 16);
            const uint32_t len = ld32(data);
            const float c = d * __ldg(x + vid) / (float)total;
            // entries: words [hdr, hdr + len) (unweighted) or the even words of [2, 2 + 2 len)
            constexpr uint32_t hdr = rec_hdr_words(kWeighted);
            const uint32_t wend = hdr + (len << wshift), qend = (wend + 3) >> 2;
            for (uint32_t qb = tid; qb < qend; qb += T * kPrUnroll) {
                uint4 v[kPrUnroll];
#pragma unroll
                for (int u = 0; u < kPrUnroll; ++u) {
                    const uint32_t q = qb + u * T;
                    if (q < qend) v[u] = ld_stream_v4(q4 + q, pol);
                }
#pragma unroll
                for (int u = 0; u < kPrUnroll; ++u) {
                    const uint32_t q = qb + u * T;
                    if (q >= qend) break;
#pragma unroll
                    for (int k = 0; k < 4; ++k) {
                        const uint32_t w = 4 * q + k;
                        if (w >= hdr && w < wend && !(kWeighted && (k & 1)))
                            em.edge(pr_decode<kVid>(word_of(v[u], k), ps.rvt_start), c);
                    }
                }
            }
        } else {
            const uint32_t start = ld32(end - kSpFooter - kSlotBytes);
            // Tiles of TV = VPT * T consecutive vertices.  Software pipeline over the page's
            // tiles: the slot offsets and x values of tile t+1 are loaded into registers
            // while tile t's records stream, so a tile exposes one DRAM latency (its
            // records) instead of three in a row (offsets, then x, then records) -- on
            // low-degree pages a tile's records are only a few KB, so latencies, not
            // bytes, set the walk's time.
            constexpr uint32_t TV = (uint32_t)T * VPT;
            uint32_t r_off[VPT], r_nxt = 0;
            float r_x[VPT];
            auto prefetch = [&](uint32_t t0) {
                const uint32_t nv = min(TV, nslots - t0);
#pragma unroll
                for (int k = 0; k < VPT; ++k) {
                    const uint32_t i = (uint32_t)tid + (uint32_t)k * T;
                    if (i < nv) {
                        const uint8_t* slot = end - kSpFooter - kSlotBytes * (uint64_t)(t0 + i + 1);
                        r_off[k] = ld_stream_u32(slot + 4, pol);
                        r_x[k] = ld_stream_f32(x + start + t0 + i, pol);
                        if (i == nv - 1)              // end of the tile's last record: the next slot's offset
                            r_nxt = t0 + nv < nslots ? ld_stream_u32(slot - kSlotBytes + 4, pol) : 0xFFFFFFFFu;
                    }
                }
            };
            prefetch(0);
            for (uint32_t t0 = 0; t0 < nslots; t0 += TV) {
                const uint32_t nv = min(TV, nslots - t0);
#pragma unroll
                for (int k = 0; k < VPT; ++k) {
                    const uint32_t i = (uint32_t)tid + (uint32_t)k * T;
                    if (i < nv) {
                        sm.off[i] = r_off[k] >> 2;
                        if (i == nv - 1)              // the page's last record ends after its own length
                            sm.off[nv] = r_nxt != 0xFFFFFFFFu ? r_nxt >> 2
                                                              : (r_off[k] >> 2) + rec_hdr_words(kWeighted) +
                                                                    (ld32(data + r_off[k]) << wshift);
                    }
                }
                __syncthreads();
#pragma unroll
                for (int k = 0; k < VPT; ++k) {
                    const uint32_t i = (uint32_t)tid + (uint32_t)k * T;
                    if (i < nv) {
                        const uint32_t deg = (sm.off[i + 1] - sm.off[i] - rec_hdr_words(kWeighted)) >> wshift;
                        float c = 0.f;
                        // dangling mass (R3); a routed rank counts only its own WA range (under
                        // S_BCAST every rank sees every page)
                        if (deg == 0 && ((kMode != kRoute && kMode != kRouteHash) ||
                                         (uint64_t)(start + t0 + i) - rp.lo < rp.hi - rp.lo))
                            dang += (double)r_x[k];
                        else c = d * r_x[k] / (float)deg;
                        sm.c[i] = c;
                    }
                }
                if (t0 + TV < nslots) prefetch(t0 + TV);
                __syncthreads();
                // the tile's record region, 16-byte evict_first loads, kPrUnroll in flight per
                // thread (coalesced: lane-consecutive groups); the owner of each 16-byte group by
                // a binary search over the tile's offsets, then record by record.  (Measured on
                // RMAT-27 and rejected: 4 consecutive groups per thread with one search per 16
                // words, 14.4 vs 11.5 ms -- uncoalesced loads; warp windows with record-start
                // masks instead of the searches, 10.82 vs 10.78 ms; a 64-cell coarse index per
                // tile narrowing each search to one cell's records, 10.90 ms -- the searches'
                // stalls are not what bounds the kernel, its L2 reductions are.)
                const uint32_t W0 = sm.off[0], W1 = sm.off[nv];
                const uint32_t qbeg = W0 >> 2, qend = (W1 + 3) >> 2;
                for (uint32_t qb = qbeg + tid; qb < qend; qb += T * kPrUnroll) {
                    uint4 v[kPrUnroll];
#pragma unroll
                    for (int u = 0; u < kPrUnroll; ++u) {
                        const uint32_t q = qb + u * T;
                        if (q < qend) v[u] = ld_stream_v4(q4 + q, pol);
                    }
#pragma unroll
                    for (int u = 0; u < kPrUnroll; ++u) {
                        const uint32_t q = qb + u * T;
                        if (q >= qend) break;
                        const uint32_t w0 = 4 * q;
                        uint32_t lo = 0, hi = nv;               // off[lo] <= max(w0, W0) < off[hi]
                        while (hi - lo > 1) {
                            const uint32_t mid = (lo + hi) >> 1;
                            if (sm.off[mid] <= w0) lo = mid; else hi = mid;
                        }
                        uint32_t j = lo, cur = sm.off[j], nxt = sm.off[j + 1];
#pragma unroll
                        for (int k = 0; k < 4; ++k) {
                            const uint32_t w = w0 + k;
                            if (w < W0 || w >= W1) continue;
                            while (w >= nxt) {
                                ++j;
                                cur = nxt;
                                nxt = sm.off[j + 1];
                            }
                            // entries: rel >= 1 (unweighted); weighted records (sz, 0, (adj, w) pairs):
                            // the even rel >= 2 (records are 8-byte aligned)
                            const uint32_t rel = w - cur;
                            if (kWeighted ? (rel < 2 || (rel & 1)) : rel == 0) continue;
                            em.edge(pr_decode<kVid>(word_of(v[u], k), ps.rvt_start), sm.c[j]);
                        }
                    }
                }
                __syncthreads();
            }
        }
        em.flush();
    }
    __syncthreads();
    if (kMode == kHash) {
        for (uint32_t i = tid; i < kHotSlots; i += T) {
            const uint32_t k = hkeys[i];
            const float v = hacc[i];
            if (k != kHotEmpty && v != 0.f) atomicAdd(acc + k, v);
        }
    } else if (kMode == kRouteHash) {      // hot partials to this rank's WA or to their owners
        for (uint32_t i = tid; i < kHotSlots; i += T) {
            const uint32_t k = hkeys[i];
            const float v = hacc[i];
            if (k != kHotEmpty && v != 0.f) em.cold(k, v);
        }
    } else if (kMode == kRoute) {
        for (uint32_t i = tid; i < n_hot; i += T) {
            const float v = hacc[i];
            if (v == 0.f) continue;
            if ((uint64_t)i >= rp.lo && (uint64_t)i < rp.hi) atomicAdd(rp.acc_loc + i, v);
            else if (rp.direct) atomicAdd(rp.peer_acc[route_owner(rp.ro, i)] + i, v);
            else if (!rp.drop_remote) atomicAdd(rp.hot_out + i, v);
        }
    } else {
        for (uint32_t i = tid; i < n_hot; i += T) {
            const float v = hacc[i];
            if (v != 0.f) atomicAdd(acc + i, v);
        }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) dang += __shfl_down_sync(0xFFFFFFFFu, dang, o);
    if ((tid & 31) == 0 && dang != 0.0) atomicAdd(dang_out, dang);
    if ((kMode == kRoute || kMode == kRouteHash) && rp.direct) __threadfence_system();   // peer atomics first
}

// Plain push PageRank (Alg 4/5: c = d x[u] / deg(u), one red.add per edge, no
// hot set) on the generic page engine, for the micro-level comparison of App E
// (GTS_MICRO_EDGE / VERTEX / HYBRID / TILE).  Same arguments as pr_scatter_kernel.
template <bool W>
struct PrMicroOp {
    static constexpr bool kReadWeights = false;
    static constexpr bool kWeighted = W;
    const float* x;
    float* acc;
    float d;
    double dang;
    __device__ const uint32_t* frontier() const { return nullptr; }
    __device__ bool select(uint32_t) { return true; }
    __device__ uint32_t payload(uint32_t v, uint32_t deg) {
        const float xv = __ldg(x + v);
        if (deg == 0) {
            dang += xv;
            return 0u;
        }
        return __float_as_uint(d * xv / (float)deg);
    }
    __device__ bool select_lp(uint32_t vid, uint32_t total, uint32_t, uint32_t& pl) {
        pl = __float_as_uint(d * __ldg(x + vid) / (float)total);   // R4: total out-degree
        return true;
    }
    __device__ __forceinline__ void edges(const uint32_t* dst, const uint32_t*, const uint32_t* pl, const uint32_t*,
                                          const bool* valid) {
#pragma unroll
        for (int q = 0; q < kEdgesPerThread; ++q)
            if (valid[q]) atomicAdd(acc + dst[q], __uint_as_float(pl[q]));
    }
    __device__ void end_page() {}
};

template <bool W, int M>
__global__ void __launch_bounds__(kThreads, 2)
pr_micro_kernel(PageSet ps, const float* __restrict__ x, float* acc, const uint32_t* __restrict__, float d,
                double* dang_out, uint32_t* work_ctr, uint32_t, const RouteParams) {
    __shared__ TileSmem sm;
    PrMicroOp<W> op{x, acc, d, 0.0};
    expand_pages<PrMicroOp<W>, M>(ps, op, sm, work_ctr);
    double v = op.dang;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_down_sync(0xFFFFFFFFu, v, o);
    if ((threadIdx.x & 31) == 0 && v != 0.0) atomicAdd(dang_out, v);
}

// x^0 = 1/n over the rank's RA (R2), acc = 0 over its WA
__global__ void pr_init_kernel(float* x, uint64_t xn, float* acc, uint64_t an, float v0) {
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < xn || i < an; i += stride) {
        if (i < xn) x[i] = v0;
        if (i < an) acc[i] = 0.f;
    }
}

// x_v <- (1-d)/n + d*D/n + acc_v ; acc_v <- 0  for v in [lo, hi) (float4 vectorised where aligned).
// x and acc are indexed by absolute ID (a Strategy-S rank passes biased pointers to its range).
__global__ void pr_finish_kernel(float* x, float* acc, uint64_t n, uint64_t lo, uint64_t hi, double d,
                                 const double* dang, double* dang_reset, int uniform) {
    const double D = *dang;
    const float base = (float)((1.0 - d) / (double)n + (uniform ? d * D / (double)n : 0.0));
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    const uint64_t t0 = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    // float4 body where x + v and acc + v share their 16-byte phase (a biased pointer of a
    // Strategy-S range need not be 16-byte aligned at a multiple of 4); scalar head and tail
    const uintptr_t px = (uintptr_t)(x + lo), pa = (uintptr_t)(acc + lo);
    const uint64_t len = hi - lo;
    const uint64_t head = ((px ^ pa) & 15u) ? len : std::min<uint64_t>(len, ((16u - (px & 15u)) & 15u) / 4u);
    const uint64_t nvec = (len - head) / 4;
    float4* x4 = reinterpret_cast<float4*>(x + lo + head);
    float4* acc4 = reinterpret_cast<float4*>(acc + lo + head);
    const float4 z = make_float4(0.f, 0.f, 0.f, 0.f);
    // four float4 loads in flight per thread before their stores (one in flight measured
    // 0.52 ms per RMAT-27 iteration, 48% of the copy peak)
    constexpr int U = 4;
    for (uint64_t i0 = t0; i0 < nvec; i0 += U * stride) {
        float4 a[U];
#pragma unroll
        for (int u = 0; u < U; ++u)
            if (i0 + u * stride < nvec) a[u] = acc4[i0 + u * stride];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const uint64_t i = i0 + u * stride;
            if (i < nvec) {
                x4[i] = make_float4(base + a[u].x, base + a[u].y, base + a[u].z, base + a[u].w);
                acc4[i] = z;
            }
        }
    }
    const uint64_t tail0 = head + 4 * nvec;
    for (uint64_t k = t0; k < head + (len - tail0); k += stride) {     // head [0, head) and tail [tail0, len)
        const uint64_t i = lo + (k < head ? k : tail0 + (k - head));
        x[i] = base + acc[i];
        acc[i] = 0.f;
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) *dang_reset = 0.0;
}

// owner side of the routed scatter: acc[dst] += value for every received (dst, value)
struct PrRecv {
    const uint2* recv;
    uint64_t off[kMaxRanks];
    const unsigned long long* cnt;
    int nranks;
};

__global__ void pr_route_apply_kernel(PrRecv rv, float* acc) {
    for (int p = 0; p < rv.nranks; ++p) {
        const uint64_t c = rv.cnt[p];
        for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < c; i += (uint64_t)gridDim.x * blockDim.x) {
            const uint2 e = rv.recv[rv.off[p] + i];
            atomicAdd(acc + e.x, __uint_as_float(e.y));
        }
    }
}

enum { kBufX = 20, kBufAcc, kBufDang, kBufPrCtr, kBufPrHot = 24, kBufPrList = 28 };
constexpr int kBufPrMulti = 300;   // multi-rank slot i: kBufPrMulti + 8 i + k
constexpr int kBufPrRoute = 120;   // route buffers

}  // namespace gts

using namespace gts;

namespace {

struct PrSlot {
    int r = 0;
    uint64_t lo = 0, hi = 0;              // WA range this rank finishes
    float *x = nullptr, *acc = nullptr;   // absolute-index (biased) pointers
    float* hot = nullptr;                 // Strategy-S: dense partials [0, n_hot) of remote hot vertices
    float* acc2 = nullptr;                // GTS_ROUTE_PEER: the second WA buffer (odd iterations)
    std::array<float*, kMaxRanks> peer[2] = {};   // GTS_ROUTE_PEER: every owner's acc / acc2 (biased)
    double* dang = nullptr;               // [2] dangling-mass accumulators (ping-pong)
    std::vector<uint32_t> pages;          // host page ids (ascending)
    const uint32_t* d_pages = nullptr;    // device page ids (nullptr: all local pages in order)
};

}  // namespace

extern "C" int gts_pagerank(gts_context* c, const gts_graph* g, uint32_t iters, double damping, uint32_t dangling,
                            const gts_run_config* cfg, float* rank_out, gts_run_stats* st) {
    clear_error();
    const double t_start = now_s();
    gts_run_config rc;
    GTS_TRY(validate_common(c, g, cfg, &rc));
    if (!rank_out) return fail(GTS_EINVAL, "NULL output");
    if (!(damping >= 0.0 && damping <= 1.0)) return fail(GTS_EINVAL, "damping must be in [0,1]");
    if (dangling > GTS_DANGLING_DROP) return fail(GTS_EINVAL, "unknown dangling mode %u", dangling);
    Ranks R;
    GTS_TRY(make_ranks(c, rc, &R));
    const uint64_t n = g->n;
    const int N = R.world, L = R.nloc;
    const uint32_t strat = R.world > 1 ? rc.strategy : GTS_STRATEGY_P;
    const bool route = strat == GTS_STRATEGY_S, bcast = strat == GTS_STRATEGY_S_BCAST;
    // GTS_ROUTE_PEER: the scatter adds remote updates straight into their owner's WA over
    // peer memory (fused scatter + exchange); acc is double-buffered so that no rank adds
    // into a buffer its owner is still finishing (iteration t adds into acc[t & 1])
    const bool peer = route && (rc.flags & GTS_ROUTE_PEER);
    // (Fusing iteration t's finish into iteration t+1's read of x -- x_u = base(D_t) + acc_t[u],
    // acc double-buffered, the buffer just read cleared by a memset -- measured on RMAT-27: call
    // 113.9 vs 115.0 ms but the scatter 11.03 vs 10.88 ms; not adopted.)
    const bool sharded = route || bcast;     // WA range-partitioned (the kRoute scatter)
    const bool streamed = choose_streamed(c, g, rc, route ? 8 * n / N + 4 * kHotDenseBig : 8 * n);
    double upload_s = 0;
    GTS_TRY(ensure_graph(c, g, rc.strategy, !streamed, &upload_s));
    const bool timing = rc.flags & GTS_RUN_TIMING;
    const uint32_t micro = (rc.flags & GTS_MICRO_MASK) >> 8;
    if (micro > (GTS_MICRO_TILE >> 8)) return fail(GTS_EINVAL, "unknown GTS_MICRO value");
    cudaStream_t s = c->stream;
    const int eg = c->num_sms * 4;
    // scatter variant: degree-ordered graphs the dense hot set held by one 1024-thread CTA per SM
    // (53,248 floats; two 512-thread CTAs with 24,576 each measured 3% slower on RMAT-27);
    // natural-order graphs the hash table; Strategy-S / S_BCAST the dense set with the owner test
    const int mode = sharded ? (g->ordered ? kRoute : kRouteHash) : (g->ordered ? kDense : kHash);
    const void* kern;
    size_t dyn;
    int threads;
    uint32_t n_hot;
    if (micro) {
        // App E comparison: the generic engine with plain REDs (TILE = 4 -> engine mode kMicroTile)
        static const void* mk[2][4] = {
            {(const void*)pr_micro_kernel<false, kMicroTile>, (const void*)pr_micro_kernel<false, kMicroEdge>,
             (const void*)pr_micro_kernel<false, kMicroVertex>, (const void*)pr_micro_kernel<false, kMicroHybrid>},
            {(const void*)pr_micro_kernel<true, kMicroTile>, (const void*)pr_micro_kernel<true, kMicroEdge>,
             (const void*)pr_micro_kernel<true, kMicroVertex>, (const void*)pr_micro_kernel<true, kMicroHybrid>}};
        kern = mk[g->weighted ? 1 : 0][micro & 3];
        dyn = 0;
        threads = kThreads;
        n_hot = 0;
    } else {
        // template instance: <weighted, mode, threads, CTAs/SM, hot set, vertices per thread, VID32 entries>
        const bool vid = g->entry_encoding == GTS_ENTRY_VID32;
#define GTS_PRK(W, M, TT, MB, HH, V) (vid ? (const void*)pr_scatter_kernel<W, M, TT, MB, HH, V, true> \
                                          : (const void*)pr_scatter_kernel<W, M, TT, MB, HH, V, false>)
        if (mode == kHash) {
            kern = g->weighted ? GTS_PRK(true, kHash, kThreads, 2, 0, 1) : GTS_PRK(false, kHash, kThreads, 2, 0, 1);
            dyn = pr_dyn_smem<kHash, 0>();
            threads = kThreads;
            n_hot = 0;
        } else if (mode == kRouteHash) {
            kern = g->weighted ? GTS_PRK(true, kRouteHash, kThreads, 2, 0, 1)
                               : GTS_PRK(false, kRouteHash, kThreads, 2, 0, 1);
            dyn = pr_dyn_smem<kRouteHash, 0>();
            threads = kThreads;
            n_hot = 0;
        } else {
            // 2048-vertex tiles (two vertices per thread): RMAT-27 scatter 10.8 ms against 11.3 ms
            // for 1024-vertex tiles and 11.1 ms for 4096-vertex tiles with a 49,152-float hot set
            const int m = mode == kRoute ? kRoute : kDense;
            if (m == kRoute)
                kern = g->weighted ? GTS_PRK(true, kRoute, 1024, 1, kHotDenseBig, kPrVpt)
                                   : GTS_PRK(false, kRoute, 1024, 1, kHotDenseBig, kPrVpt);
            else
                kern = g->weighted ? GTS_PRK(true, kDense, 1024, 1, kHotDenseBig, kPrVpt)
                                   : GTS_PRK(false, kDense, 1024, 1, kHotDenseBig, kPrVpt);
            dyn = pr_dyn_smem<kDense, kHotDenseBig>();
            threads = 1024;
            n_hot = (uint32_t)std::min<uint64_t>(n, kHotDenseBig);
        }
#undef GTS_PRK
    }
    GTS_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)dyn));
    int grid = 0;
    GTS_TRY(sms_grid(c, kern, threads, dyn, &grid));
    const uint32_t hybrid_deg = rc.hybrid_deg ? rc.hybrid_deg : 8u;

    // ---- the ranks of this call and their WA (a1) ----
    std::vector<int32_t> owner;
    std::vector<uint64_t> vr;
    partition(g, strat, N, owner, vr);
    std::vector<PrSlot> S(L);
    uint64_t wa_bytes = 0;
    for (int i = 0; i < L; ++i) {
        PrSlot& m = S[i];
        m.r = R.rank(i);
        if (R.virt) {
            for (uint64_t j = 0; j < g->num_pages; ++j)
                if (bcast || owner[j] == m.r) m.pages.push_back((uint32_t)j);
            uint32_t* dp;
            GTS_TRY(c->buf(kBufPrMulti + 8 * i, std::max<size_t>(m.pages.size(), 1) * 4, (void**)&dp));
            if (!m.pages.empty())
                GTS_CUDA(cudaMemcpyAsync(dp, m.pages.data(), m.pages.size() * 4, cudaMemcpyHostToDevice, s));
            m.d_pages = dp;
        } else {
            m.pages = c->dg.h_local_list;
            m.d_pages = (c->dg.all_local && !streamed) ? nullptr : c->dg.local_list;
        }
        m.lo = sharded ? vr[m.r] : 0;
        m.hi = sharded ? vr[m.r + 1] : n;
        // RA x: the rank's sources (S: its own range; P / S_BCAST: every vertex);
        // WA acc: its range (S, S_BCAST) or the full replica (P)
        const uint64_t xlo = route ? m.lo : 0, xn = route ? m.hi - m.lo : n;
        const uint64_t alo = sharded ? m.lo : 0, an = sharded ? m.hi - m.lo : n;
        float *xb, *ab;
        GTS_TRY(c->buf(L == 1 ? kBufX : kBufPrMulti + 8 * i + 1, std::max<uint64_t>(xn, 1) * 4, (void**)&xb));
        GTS_TRY(c->buf(L == 1 ? kBufAcc : kBufPrMulti + 8 * i + 2, std::max<uint64_t>(an, 1) * 4, (void**)&ab));
        GTS_TRY(c->buf(L == 1 ? kBufDang : kBufPrMulti + 8 * i + 3, 2 * sizeof(double), (void**)&m.dang));
        m.x = xb - xlo;
        m.acc = ab - alo;
        if (route && !peer) GTS_TRY(c->buf(kBufPrMulti + 8 * i + 4, std::max<uint32_t>(n_hot, 1) * 4, (void**)&m.hot));
        if (peer) {
            float* ab2;
            GTS_TRY(c->buf(kBufPrMulti + 8 * i + 5, std::max<uint64_t>(an, 1) * 4, (void**)&ab2));
            GTS_CUDA(cudaMemsetAsync(ab2, 0, std::max<uint64_t>(an, 1) * 4, s));
            m.acc2 = ab2 - alo;
        }
        if (i == 0) wa_bytes = (xn + an * (peer ? 2 : 1)) * 4 + (route && !peer ? (uint64_t)n_hot * 4 : 0);
        pr_init_kernel<<<eg, 256, 0, s>>>(xb, xn, ab, an, (float)(1.0 / (double)n));
        GTS_CUDA(cudaMemsetAsync(m.dang, 0, 2 * sizeof(double), s));
        if (m.hot) GTS_CUDA(cudaMemsetAsync(m.hot, 0, std::max<uint32_t>(n_hot, 1) * 4, s));
    }
    uint32_t* ctr;
    GTS_TRY(c->buf(kBufPrCtr, 4, (void**)&ctr));
    Route rt;
    if (peer) {                                  // map every owner's two WA buffers
        for (int k = 0; k < 2; ++k) {
            std::vector<void*> base(L);
            for (int i = 0; i < L; ++i) base[i] = (k ? S[i].acc2 : S[i].acc) + S[i].lo;
            std::vector<std::array<void*, kMaxRanks>> pm;
            GTS_TRY(R.peer_map(base.data(), pm));
            for (int i = 0; i < L; ++i)
                for (int q = 0; q < N; ++q) S[i].peer[k][q] = static_cast<float*>(pm[i][q]) - vr[q];
        }
        GTS_TRY(R.barrier());                    // every owner's buffers are zero before anyone adds
    } else if (route) {
        std::vector<std::vector<uint32_t>> pl(L);
        std::vector<const uint32_t*> dpl(L);
        for (int i = 0; i < L; ++i) {
            pl[i] = S[i].pages;
            dpl[i] = S[i].d_pages;
        }
        std::vector<std::array<uint64_t, kMaxRanks>> cap;
        GTS_TRY(route_capacities(c, g, R, rc, streamed, pl, dpl.data(), vr, n_hot, cap));
        GTS_TRY(route_setup(c, R, cap, 8, kBufPrRoute, rt));
    }
    GTS_CUDA(cudaStreamSynchronize(s));      // host page lists are read by the copies above
    // L2 persistence for the hot head of WA: on a degree-ordered graph the most updated
    // entries are acc[0, W) (gts_run_config.l2_persist_mib, default 96 MiB, clipped to the
    // device's persisting-L2 limit)
    const bool persist = g->ordered && !sharded && l2_persist_mib(rc) > 0;
    uint64_t launches = L, main_launches = 0;
    SweepStats ss;
    const float dmp = (float)damping;
    const uint32_t* hk = c->dg.hot_keys;
    auto scatter = [&](PrSlot& m, const PageSet& ps, int gcap, double* D, const RouteParams& rp) -> int {
        GTS_CUDA(cudaMemsetAsync(ctr, 0, 4, s));
        std::pair<cudaEvent_t, cudaEvent_t> e2;
        if (timing) { e2 = c->t_main.next(); cudaEventRecord(e2.first, s); }
        PageSet p2 = ps;
        p2.hybrid_deg = hybrid_deg;
        const float* xr = m.x;
        float* ar = m.acc;
        void* args[] = {(void*)&p2, (void*)&xr, (void*)&ar, (void*)&hk, (void*)&dmp, (void*)&D, (void*)&ctr,
                        (void*)&n_hot, (void*)&rp};
        cudaLaunchConfig_t lc;
        std::memset(&lc, 0, sizeof(lc));
        lc.gridDim = dim3(std::min(grid, gcap));
        lc.blockDim = dim3(threads);
        lc.dynamicSmemBytes = dyn;
        lc.stream = s;
        GTS_CUDA(cudaLaunchKernelExC(&lc, kern, args));
        if (timing) cudaEventRecord(e2.second, s);
        GTS_CUDA(cudaGetLastError());
        ++main_launches;
        return GTS_OK;
    };
    for (uint32_t it = 0; it < iters; ++it) {
        const int cur_d = it & 1;
        if (route && !peer) GTS_CUDA(cudaMemsetAsync(rt.d_scnt, 0, (size_t)L * kMaxRanks * 8, s));
        for (int i = 0; i < L; ++i) {           // ---- a7 / a8: the scatter over this rank's pages ----
            PrSlot& m = S[i];
            RouteParams rp;
            std::memset(&rp, 0, sizeof(rp));
            rp.acc_loc = (peer && (it & 1)) ? m.acc2 : m.acc;
            rp.hot_out = m.hot;
            rp.lo = m.lo;
            rp.hi = m.hi;
            rp.drop_remote = bcast ? 1 : 0;
            if (peer) {
                rp.direct = 1;
                for (int q = 0; q <= N; ++q) rp.ro.vr[q] = vr[q];
                rp.ro.nranks = N;
                for (int q = 0; q < N; ++q) rp.peer_acc[q] = m.peer[it & 1][q];
            } else if (route) {
                rp.ro.send = rt.send[i];
                rp.ro.cnt = rt.d_scnt + (size_t)i * kMaxRanks;
                rp.ro.ovf = rt.d_ovf + i;
                for (int q = 0; q <= N; ++q) rp.ro.vr[q] = vr[q];
                for (int q = 0; q < N; ++q) {
                    rp.ro.off[q] = rt.soff[i][q];
                    rp.ro.cap[q] = rt.scap[i][q];
                }
                rp.ro.nranks = N;
            }
            if (persist) GTS_TRY(persist_window(c, s, m.acc, std::min<size_t>(l2_persist_mib(rc) << 20, n * 4)));
            std::vector<uint32_t> hl(m.pages);
            GTS_TRY(sweep_pages(c, g, rc, streamed, &hl, m.d_pages, (uint32_t)hl.size(), nullptr,
                                [&](const PageSet& ps, int gcap) -> int {
                                    return scatter(m, ps, gcap, m.dang + cur_d, rp);
                                }, &ss));
        }
        // ---- a12: merge ----
        std::pair<cudaEvent_t, cudaEvent_t> ev;
        if (timing) { ev = c->t_merge.next(); cudaEventRecord(ev.first, s); }
        if (N > 1) {
            std::vector<void*> db(L);
            for (int i = 0; i < L; ++i) db[i] = S[i].dang + cur_d;
            if (strat == GTS_STRATEGY_P) {      // every replica receives the full sum
                std::vector<void*> ab(L);
                for (int i = 0; i < L; ++i) ab[i] = S[i].acc;
                GTS_TRY(R.allreduce(ab.data(), n, kCF32, kCSum));
            } else if (route && !peer) {        // hot partials to their owners, then the routed pairs
                std::vector<float*> part(L), dst(L);
                for (int i = 0; i < L; ++i) {
                    part[i] = S[i].hot;
                    dst[i] = S[i].acc;
                }
                GTS_TRY(R.reduce_to_owners(part.data(), dst.data(), vr, n_hot));
                GTS_TRY(R.route_exchange(rt));
                for (int i = 0; i < L; ++i) {
                    PrRecv rv{};
                    rv.recv = reinterpret_cast<const uint2*>(rt.recv[i]);
                    for (int q = 0; q < N; ++q) rv.off[q] = rt.roff[i][q];
                    rv.cnt = rt.d_rcnt + (size_t)i * kMaxRanks;
                    rv.nranks = N;
                    pr_route_apply_kernel<<<eg, 256, 0, s>>>(rv, S[i].acc);
                    ++launches;
                }
            }
            GTS_TRY(R.allreduce(db.data(), 1, kCF64, kCSum));   // dangling mass D (R3)
        }
        if (timing) { cudaEventRecord(ev.second, s); ev = c->t_finish.next(); cudaEventRecord(ev.first, s); }
        // ---- a9: fused damping / dangling / swap over each rank's range ----
        for (PrSlot& m : S) {
            // (GTS_ROUTE_PEER: the D all-reduce above is also the barrier after every rank's peer adds)
            pr_finish_kernel<<<2 * eg, 256, 0, s>>>(m.x, (peer && (it & 1)) ? m.acc2 : m.acc, n, m.lo, m.hi, damping,
                                                     m.dang + cur_d,
                                                     m.dang + (cur_d ^ 1), dangling == GTS_DANGLING_UNIFORM ? 1 : 0);
            ++launches;
        }
        if (bcast) {                            // every rank reads every source's RA next iteration
            std::vector<void*> xb(L);
            for (int i = 0; i < L; ++i) xb[i] = S[i].x;
            GTS_TRY(R.gather_ranges(xb.data(), vr, 4));
        }
        if (timing) cudaEventRecord(ev.second, s);
        GTS_CUDA(cudaGetLastError());
    }
    if (route && !peer) {
        bool ovf = false;
        GTS_TRY(R.route_overflow(rt, &ovf));
        if (ovf) return fail(GTS_ECUDA, "Strategy-S route region overflow (capacity count mismatch)");
    }
    if (persist) GTS_TRY(persist_window(c, s, nullptr, 0));
    // ---- a13: the result in one full array ----
    float* res = S[0].x;
    if (route) {
        GTS_TRY(c->buf(kBufPrMulti + 7, n * 4, (void**)&res));
        std::vector<void*> full(L, res);
        for (PrSlot& m : S)
            if (m.hi > m.lo)
                GTS_CUDA(cudaMemcpyAsync(res + m.lo, m.x + m.lo, (m.hi - m.lo) * 4, cudaMemcpyDeviceToDevice, s));
        GTS_TRY(R.gather_ranges(full.data(), vr, 4));
    }
    GTS_CUDA(cudaGetLastError());
    GTS_TRY(deliver(c, g, reinterpret_cast<const uint32_t*>(res), rank_out, rc.out_location, false));
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
        uint64_t pages = 0;
        for (PrSlot& m : S) pages += m.pages.size();
        st->pages_processed = pages * iters;
        st->h2d_bytes = ss.h2d_bytes;
        st->edges_traversed = (bcast ? g->m * (uint64_t)L : g->m * (uint64_t)L / (uint64_t)N) * iters;
        st->nccl_bytes = R.bytes;
        st->launches = launches + main_launches;
        st->main_kernel_launches = main_launches;
        st->levels_or_iters = iters;
        st->wa_bytes = wa_bytes;
        st->routed_msgs = rt.sent_msgs;
    } else if (timing) {
        c->t_main.sum_s();
        c->t_merge.sum_s();
        c->t_finish.sum_s();
        c->t_h2d.sum_s();
    }
    return GTS_OK;
}
