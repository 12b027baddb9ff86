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

#include <cstdlib>
#include <cstring>

#include "expand.cuh"
#include "memops.cuh"
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
enum PrMode : int { kHash = 0, kDense = 1, kRoute = 2 };

constexpr int kMaxRanks = 8;

struct RouteParams {
    float* acc_loc;                    // local WA: acc_loc[v - lo]
    float* hot_out;                    // [n_hot] hot partials of vertices outside [lo, hi)
    uint2* send;                       // (dst, float bits) pairs, peer p's region at send_off[p]
    uint32_t* send_cnt;                // [nranks] pairs appended per peer
    uint32_t* overflow;                // set if a peer region is full (capacity is an upper bound)
    uint64_t vr[kMaxRanks + 1];        // WA ranges: rank p owns [vr[p], vr[p+1])
    uint32_t send_off[kMaxRanks];
    uint32_t send_cap[kMaxRanks];
    uint64_t lo, hi;
    int nranks;
    int drop_remote;                   // paper-literal Strategy-S (broadcast pages): ignore remote updates
};

__device__ __forceinline__ int route_owner(const RouteParams& rp, uint32_t v) {
    int p = 0;
    while (p < rp.nranks - 1 && (uint64_t)v >= rp.vr[p + 1]) ++p;
    return p;
}

// append (dst, c) to the owner's buffer; lanes of a warp bound for the same
// owner share one atomic on its counter
__device__ __forceinline__ void route_push(const RouteParams& rp, uint32_t dst, float c) {
    const int p = route_owner(rp, dst);
    const uint32_t active = __activemask();
    const uint32_t peers = __match_any_sync(active, p);
    const int lane = threadIdx.x & 31;
    const int leader = __ffs(peers) - 1;
    uint32_t base = 0;
    if (lane == leader) base = atomicAdd(rp.send_cnt + p, (uint32_t)__popc(peers));
    base = __shfl_sync(peers, base, leader);
    const uint32_t slot = base + __popc(peers & ((1u << lane) - 1u));
    if (slot < rp.send_cap[p]) rp.send[rp.send_off[p] + slot] = make_uint2(dst, __float_as_uint(c));
    else *rp.overflow = 1u;
}

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
            else if ((uint64_t)dst >= rp->lo && (uint64_t)dst < rp->hi) atomicAdd(rp->acc_loc + (dst - rp->lo), c);
            else if (!rp->drop_remote) route_push(*rp, dst, c);
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
        else atomicAdd(acc + dst, c);                   // REDG.E.ADD.F32 (result unused)
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
    return kMode == kHash ? kHotSlots * (sizeof(uint32_t) + sizeof(float)) : H * sizeof(float);   // kDense, kRoute
}

// dense hot-set sizes: 512-thread CTAs (2 per SM) hold kHotDense floats each;
// 1024-thread CTAs (1 per SM) hold kHotDenseBig
constexpr uint32_t kHotDenseBig = 53248;

__device__ __forceinline__ uint32_t pr_decode(uint32_t e, uint32_t enc, const uint32_t* rvt) {
    return enc == GTS_ENTRY_VID32 ? e : __ldg(rvt + (e >> 16)) + (e & 0xFFFFu);
}

// K_PR_SP / K_PR_LP (Alg 4/5) for a persistent CTA of T threads.  The record
// region of a tile of T consecutive vertices is one contiguous word range
// (records are packed in VID order from offset 0), streamed with 16-byte
// evict_first loads, kPrUnroll in flight per thread; the owner of each 4-word
// group is found by a binary search over the tile's record offsets.
template <bool kWeighted, int kMode, int T, int kMinBlocks, uint32_t H>
__global__ void __launch_bounds__(T, kMinBlocks)
pr_scatter_kernel(PageSet ps, const float* __restrict__ x, float* acc, const uint32_t* __restrict__ hot_keys,
                  float d, double* dang_out, uint32_t* work_ctr, uint32_t n_hot, const RouteParams rp) {
    __shared__ PrSmem<T> sm;
    extern __shared__ uint4 dyn_smem[];
    uint32_t* hkeys = reinterpret_cast<uint32_t*>(dyn_smem);
    float* hacc = kMode == kHash ? reinterpret_cast<float*>(hkeys + kHotSlots) : reinterpret_cast<float*>(dyn_smem);
    const int tid = threadIdx.x;
    if (kMode == kHash) {
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
    const uint32_t enc = ps.entry_encoding;
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
            const uint32_t wend = 1 + len, qend = (wend + 3) >> 2;
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
                        if (w >= 1 && w < wend) em.edge(pr_decode(word_of(v[u], k), enc, ps.rvt_start), c);
                    }
                }
            }
        } else {
            const uint32_t start = ld32(end - kSpFooter - kSlotBytes);
            for (uint32_t t0 = 0; t0 < nslots; t0 += T) {
                const uint32_t nv = min((uint32_t)T, nslots - t0);
                if ((uint32_t)tid < nv) {
                    const uint8_t* slot = end - kSpFooter - kSlotBytes * (uint64_t)(t0 + tid + 1);
                    sm.off[tid] = ld_stream_u32(slot + 4, pol) >> 2;
                    if ((uint32_t)tid == nv - 1) {                 // end of the tile's last record
                        if (t0 + nv < nslots) {
                            sm.off[nv] = ld_stream_u32(slot - kSlotBytes + 4, pol) >> 2;
                        } else {
                            const uint32_t o = ld_stream_u32(slot + 4, pol);
                            sm.off[nv] = (o >> 2) + 1 + (ld32(data + o) << wshift);
                        }
                    }
                }
                __syncthreads();
                if ((uint32_t)tid < nv) {
                    const uint32_t deg = (sm.off[tid + 1] - sm.off[tid] - 1) >> wshift;
                    const float xv = ld_stream_f32(x + start + t0 + tid, pol);
                    float c = 0.f;
                    // dangling mass (R3); a routed rank counts only its own WA range (under
                    // S_BCAST every rank sees every page)
                    if (deg == 0 && (kMode != kRoute || (uint64_t)(start + t0 + tid) - rp.lo < rp.hi - rp.lo))
                        dang += (double)xv;
                    else c = d * xv / (float)deg;
                    sm.c[tid] = c;
                }
                __syncthreads();
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
                            const uint32_t rel = w - cur;     // 0 = ADJLIST_SZ word; > deg = weight words
                            if (rel == 0 || rel > ((nxt - cur - 1) >> wshift)) continue;
                            em.edge(pr_decode(word_of(v[u], k), enc, ps.rvt_start), sm.c[j]);
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
    } else if (kMode == kRoute) {
        for (uint32_t i = tid; i < n_hot; i += T) {
            const float v = hacc[i];
            if (v == 0.f) continue;
            if ((uint64_t)i >= rp.lo && (uint64_t)i < rp.hi) atomicAdd(rp.acc_loc + (i - rp.lo), v);
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
}

// ---- Warp-window page walk ---------------------------------------------------
//
// The record region of a tile of T vertices is cut into 128-word windows (one
// 16-byte load per lane, 512 contiguous bytes per warp); each warp walks a
// contiguous run of windows.  The owner of every word comes from a 128-bit
// record-start mask built with four redux.or per 32 candidate slots and a
// popcount prefix, instead of a binary search per 16 bytes: the owner of word
// i is j0 + #(record starts at or before i), j0 = the last vertex starting
// before the window (carried from window to window).
template <bool kWeighted, int T, int kMinBlocks, uint32_t H>
__global__ void __launch_bounds__(T, kMinBlocks)
pr_scatter_ww_kernel(PageSet ps, const float* __restrict__ x, float* acc, float d, double* dang_out,
                     uint32_t* work_ctr, uint32_t n_hot) {
    __shared__ PrSmem<T> sm;
    extern __shared__ uint4 dyn_smem[];
    float* hacc = reinterpret_cast<float*>(dyn_smem);
    constexpr int kW = T / 32;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    for (uint32_t i = tid; i < H; i += T) hacc[i] = 0.f;
    __syncthreads();
    const uint64_t pol = policy_evict_first();
    const uint32_t count = ps.count;
    const uint32_t enc = ps.entry_encoding;
    constexpr uint32_t wshift = kWeighted ? 1 : 0;
    PrEmitter<kDense, H> em{acc, nullptr, hacc, nullptr, 0u, 0.f, false};
    double dang = 0.0;
    for (;;) {
        if (tid == 0) sm.item = atomicAdd(work_ctr, 1u);
        __syncthreads();
        const uint32_t it = sm.item;
        __syncthreads();
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
            const uint32_t wend = 1 + len, qend = (wend + 3) >> 2;
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
                        if (w >= 1 && w < wend) em.edge(pr_decode(word_of(v[u], k), enc, ps.rvt_start), c);
                    }
                }
            }
        } else {
            const uint32_t start = ld32(end - kSpFooter - kSlotBytes);
            for (uint32_t t0 = 0; t0 < nslots; t0 += T) {
                const uint32_t nv = min((uint32_t)T, nslots - t0);
                if ((uint32_t)tid < nv) {
                    const uint8_t* slot = end - kSpFooter - kSlotBytes * (uint64_t)(t0 + tid + 1);
                    sm.off[tid] = ld_stream_u32(slot + 4, pol) >> 2;
                    if ((uint32_t)tid == nv - 1) {
                        if (t0 + nv < nslots) {
                            sm.off[nv] = ld_stream_u32(slot - kSlotBytes + 4, pol) >> 2;
                        } else {
                            const uint32_t o = ld_stream_u32(slot + 4, pol);
                            sm.off[nv] = (o >> 2) + 1 + (ld32(data + o) << wshift);
                        }
                    }
                }
                __syncthreads();
                if ((uint32_t)tid < nv) {
                    const uint32_t deg = (sm.off[tid + 1] - sm.off[tid] - 1) >> wshift;
                    const float xv = ld_stream_f32(x + start + t0 + tid, pol);
                    float c = 0.f;
                    if (deg == 0) dang += (double)xv;      // dangling mass (R3)
                    else c = d * xv / (float)deg;
                    sm.c[tid] = c;
                }
                __syncthreads();
                const uint32_t W0 = sm.off[0], W1 = sm.off[nv];
                const uint32_t wbase = W0 & ~3u;
                const uint32_t nwin = (W1 - wbase + 127) >> 7;
                // contiguous run of windows per warp
                const uint32_t per = (nwin + kW - 1) / kW;
                const uint32_t wa = min(nwin, warp * per), wb = min(nwin, wa + per);
                if (wa < wb) {
                    const uint32_t base = wbase + (wa << 7);
                    // j0 = last vertex whose record starts before base (-1: none)
                    int lo = -1, hi = (int)nv;               // off[lo] < base <= off[hi]
                    while (hi - lo > 1) {
                        const int mid = (lo + hi) >> 1;
                        if (sm.off[mid] < base) lo = mid; else hi = mid;
                    }
                    int j0 = lo;
                    for (uint32_t wi = wa; wi < wb; wi += kPrUnroll) {
                        uint4 v[kPrUnroll];                  // kPrUnroll windows' loads in flight
#pragma unroll
                        for (int u = 0; u < kPrUnroll; ++u) {
                            const uint32_t q = ((wbase + ((wi + u) << 7)) >> 2) + lane;
                            v[u] = make_uint4(0u, 0u, 0u, 0u);
                            if (wi + u < wb && 4 * q < W1) v[u] = ld_stream_v4(q4 + q, pol);
                        }
#pragma unroll
                        for (int u = 0; u < kPrUnroll; ++u) {
                            if (wi + u >= wb) break;
                            const uint32_t bw = wbase + ((wi + u) << 7);
                            const uint32_t q = (bw >> 2) + lane;
                            int ns;
                            const WinMask wm = win_mask(sm.off, j0, nv, bw, ns);
                            const uint32_t mw = lane >> 3;
                            uint32_t before = 0;
#pragma unroll
                            for (int k = 0; k < 4; ++k) before += (uint32_t)k < mw ? __popc(wm.m[k]) : 0u;
                            const uint32_t mword = mw == 0 ? wm.m[0] : mw == 1 ? wm.m[1] : mw == 2 ? wm.m[2] : wm.m[3];
#pragma unroll
                            for (int k = 0; k < 4; ++k) {
                                const uint32_t w = 4 * q + k;
                                const uint32_t bpos = (4 * lane + k) & 31;
                                if (w < W0 || w >= W1 || ((mword >> bpos) & 1u)) continue;
                                const int j = j0 + (int)(before + __popc(mword & ((2u << bpos) - 1u)));
                                if (kWeighted) {
                                    const uint32_t o = sm.off[j];
                                    if (w - o > ((sm.off[j + 1] - o - 1) >> 1)) continue;   // weight words
                                }
                                em.edge(pr_decode(word_of(v[u], k), enc, ps.rvt_start), sm.c[j]);
                            }
                            j0 += ns;
                        }
                    }
                }
                __syncthreads();
            }
        }
        em.flush();
    }
    __syncthreads();
    for (uint32_t i = tid; i < n_hot; i += T) {
        const float v = hacc[i];
        if (v != 0.f) atomicAdd(acc + i, v);
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) dang += __shfl_down_sync(0xFFFFFFFFu, dang, o);
    if ((tid & 31) == 0 && dang != 0.0) atomicAdd(dang_out, dang);
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

__global__ void pr_init_kernel(float* x, float* acc, uint64_t n, float v0) {
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
        x[i] = v0;
        acc[i] = 0.f;
    }
}

// x_v <- (1-d)/n + d*D/n + acc_v ; acc_v <- 0  for v in [lo, hi) (float4 vectorised where aligned).
// Strategy-S ranks finish only their own WA range and zero the rest of acc.
__global__ void pr_finish_kernel(float* x, float* acc, uint64_t n, uint64_t lo, uint64_t hi, double d,
                                 const double* dang, double* dang_reset, int uniform, int zero_outside) {
    const double D = *dang;
    const float base = (float)((1.0 - d) / (double)n + (uniform ? d * D / (double)n : 0.0));
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    const uint64_t t0 = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const float4 z = make_float4(0.f, 0.f, 0.f, 0.f);
    uint64_t a4 = (lo + 3) / 4, b4 = hi / 4;            // aligned float4 span inside [lo, hi)
    if (b4 < a4) b4 = a4;
    float4* x4 = reinterpret_cast<float4*>(x);
    float4* acc4 = reinterpret_cast<float4*>(acc);
    for (uint64_t i = a4 + t0; i < b4; i += stride) {
        const float4 a = acc4[i];
        x4[i] = make_float4(base + a.x, base + a.y, base + a.z, base + a.w);
        acc4[i] = z;
    }
    if (t0 < 8) {                                       // unaligned head [lo, 4*a4) and tail [4*b4, hi)
        const uint64_t i = t0 < 4 ? lo + t0 : 4 * b4 + (t0 - 4);
        const bool ok = t0 < 4 ? (i < 4 * a4 && i < hi) : (i < hi && i >= 4 * a4);
        if (ok) {
            x[i] = base + acc[i];
            acc[i] = 0.f;
        }
    }
    if (zero_outside && (lo > 0 || hi < n)) {           // zero acc outside my range
        for (uint64_t i = t0; i < n; i += stride)
            if (i < lo || i >= hi) acc[i] = 0.f;
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) *dang_reset = 0.0;
}

// ---- Strategy-S with routed updates: capacity count, apply -----------------

template <bool W>
struct RouteCountOp {   // per-owner count of this rank's remote cold edges (send capacities)
    static constexpr bool kReadWeights = false;
    static constexpr bool kWeighted = W;
    const RouteParams* rp;
    uint32_t n_hot;
    uint32_t cnt[kMaxRanks];
    __device__ const uint32_t* frontier() const { return nullptr; }
    __device__ bool select(uint32_t) { return true; }
    __device__ uint32_t payload(uint32_t, uint32_t) { return 0u; }
    __device__ bool select_lp(uint32_t, uint32_t, uint32_t, uint32_t&) { return true; }
    __device__ __forceinline__ void edges(const uint32_t* dst, const uint32_t*, const uint32_t*, const uint32_t*,
                                          const bool* ok) {
#pragma unroll
        for (int q = 0; q < kEdgesPerThread; ++q) {
            const uint32_t v = dst[q];
            if (ok[q] && v >= n_hot && !((uint64_t)v >= rp->lo && (uint64_t)v < rp->hi)) {
                const int p = route_owner(*rp, v);
#pragma unroll
                for (int k = 0; k < kMaxRanks; ++k) cnt[k] += (k == p);
            }
        }
    }
    __device__ void end_page() {}
};

template <bool W>
__global__ void __launch_bounds__(kThreads, 2)
route_count_kernel(PageSet ps, const RouteParams rp, uint32_t n_hot, unsigned long long* out, uint32_t* work_ctr) {
    __shared__ TileSmem sm;
    RouteCountOp<W> op{&rp, n_hot, {0, 0, 0, 0, 0, 0, 0, 0}};
    expand_pages(ps, op, sm, work_ctr);
#pragma unroll
    for (int k = 0; k < kMaxRanks; ++k) {
        unsigned long long v = op.cnt[k];
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) v += __shfl_down_sync(0xFFFFFFFFu, v, o);
        if ((threadIdx.x & 31) == 0 && v) atomicAdd(out + k, v);
    }
}

// acc_loc[dst - lo] += val for the received (dst, val) pairs of every peer region
__global__ void route_apply_kernel(const uint2* __restrict__ pairs, const uint32_t* __restrict__ off,
                                   const uint32_t* __restrict__ cnt, int nranks, float* acc_loc, uint32_t lo) {
    for (int p = 0; p < nranks; ++p) {
        const uint32_t c = cnt[p], o = off[p];
        for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < c; i += gridDim.x * blockDim.x) {
            const uint2 e = pairs[o + i];
            atomicAdd(acc_loc + (e.x - lo), __uint_as_float(e.y));
        }
    }
}

// acc[i] += hot[i], hot[i] = 0 over [a, b)
__global__ void dense_add_kernel(float* acc, float* hot, uint64_t a, uint64_t b) {
    for (uint64_t i = a + (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < b;
         i += (uint64_t)gridDim.x * blockDim.x) {
        const float v = hot[i];
        if (v != 0.f) {
            acc[i] += v;
            hot[i] = 0.f;
        }
    }
}

// ---- Binned scatter (propagation blocking) for degree-ordered pages ---------
//
// The plain scatter issues one L2 reduction per cold edge (~1.7 G per RMAT-27
// iteration), and L2 reduction throughput (~188 G/s measured) is what bounds
// it.  The binned scatter keeps Alg 4/5's push order but defers the WA update
// (DESIGN.md section 6b):
//   phase 1 (pr_bin_kernel): the page sweep; hot destinations [0, hot) are
//     summed per CTA in shared memory as before; every other (dst, c) pair is
//     appended to the bin of dst's range: a CTA stages up to kPbStage pairs of
//     a round in shared memory, counting-sorts them by bin and writes each
//     bin's run with one global cursor bump (coalesced 8-byte pairs);
//   phase 2 (pr_apply_kernel): per (bin, chunk) work item, fine bins (ranges
//     of 2^fine_shift vertices) are summed in a shared-memory slice of WA and
//     flushed with 16-byte reductions; coarse bins (the cold tail, whose WA
//     slice stays L2-resident while its items run) take one L2 red per pair.
// Same additions per destination as Alg 4 l.16, grouped by destination range.
constexpr int kPbThreads = 512;
constexpr int kPbBlocks = 2;                                   // CTAs per SM (phase 1)
constexpr uint32_t kPbUnroll = 2;                              // 16-byte words per thread per round
constexpr uint32_t kPbStage = kPbThreads * kPbUnroll * 4;      // pairs staged per round (4096)
constexpr uint32_t kPbMaxBins = 1024;                          // two bins per thread in the scan
constexpr uint32_t kPbHot = 8192;                              // shared-memory hot set (32 KB)
constexpr uint32_t kPbFineShiftMax = 15;                       // phase-2 slice: 2^15 floats (128 KB)
constexpr int kPbWarps = kPbThreads / 32;

struct PbGeom {
    uint32_t hot;          // destinations [0, hot) use the shared-memory hot set (multiple of 4, <= kPbHot)
    uint32_t fine_shift;   // fine bins: 2^fine_shift vertices each, starting at `hot`
    uint32_t nfine;
    uint32_t coarse_shift; // coarse bins: 2^coarse_shift vertices each, starting at fine_end
    uint32_t nbins;
    uint64_t fine_end;     // hot + nfine << fine_shift
    uint64_t n;
};

__device__ __forceinline__ uint32_t pb_bin(const PbGeom& g, uint32_t v) {
    return (uint64_t)v < g.fine_end ? (v - g.hot) >> g.fine_shift
                                    : g.nfine + (uint32_t)(((uint64_t)v - g.fine_end) >> g.coarse_shift);
}

struct PbParams {
    PbGeom geo;
    uint2* pairs;                 // bin b occupies pairs[boff[b], boff[b] + cap[b])
    const uint32_t* boff;         // [nbins]
    uint32_t* cur;                // [nbins] pairs appended (phase 1), zeroed before the sweep
    unsigned long long* count;    // count mode: [nbins] pairs per bin
};

struct PbSmem {                   // dynamic shared memory after the hot set
    uint2 stage[kPbStage];
    uint16_t sbin[kPbStage];
    uint32_t hist[kPbMaxBins];
    uint32_t start[kPbMaxBins];
    uint32_t gpos[kPbMaxBins];
    uint32_t wsum[kPbWarps];
};

__device__ __forceinline__ void st_stream_v2(uint2* p, uint2 v) {
    asm volatile("st.global.cs.v2.u32 [%0], {%1,%2};" ::"l"(p), "r"(v.x), "r"(v.y) : "memory");
}

// Per-thread run combiner for hot destinations (rows are sorted, so a thread's
// consecutive edges often share a hub): one shared-memory add per run, which
// keeps a hub's fp32 sum two-level (SURVEY section 7 hard parts).
struct HotRun {
    uint32_t last;
    float sum;
    __device__ __forceinline__ void add(float* hacc, uint32_t v, float c) {
        if (v == last) {
            sum += c;
            return;
        }
        if (last != 0xFFFFFFFFu) atomicAdd(hacc + last, sum);
        last = v;
        sum = c;
    }
    __device__ __forceinline__ void flush(float* hacc) {
        if (last != 0xFFFFFFFFu) atomicAdd(hacc + last, sum);
        last = 0xFFFFFFFFu;
    }
};

constexpr uint32_t kNoEdge = 0xFFFFFFFFu;   // VIDs are < 2^32 - 1 (n <= 2^32 - 1)

// One staging round of the CTA: every thread hands in up to kPbUnroll*4 edges
// (dst[k], c[k]; dst[k] = kNoEdge: no edge).  Hot destinations go to the thread's
// run combiner; the rest are ranked per bin (shared-memory counters),
// counting-sorted into stage[] and written out bin run by bin run, one global
// cursor bump per non-empty bin.  Four barriers; all threads call.
template <bool kCount>
__device__ __forceinline__ void pb_round(const PbParams& pb, float* hacc, HotRun& hr, PbSmem& s, const uint32_t* dst,
                                         const float* c) {
    constexpr int E = kPbUnroll * 4;
    uint32_t rk[E / 2];                                // per-bin ranks, two 16-bit halves; 0xFFFF = none
#pragma unroll
    for (int k = 0; k < E; ++k) {
        uint32_t r = 0xFFFFu;
        if (dst[k] != kNoEdge) {
            if (dst[k] < pb.geo.hot) {
                if (!kCount) hr.add(hacc, dst[k], c[k]);
            } else {
                r = atomicAdd(s.hist + pb_bin(pb.geo, dst[k]), 1u);
            }
        }
        if (k & 1) rk[k >> 1] |= r << 16;
        else rk[k >> 1] = r;
    }
    if (kCount) return;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    __syncthreads();
    // exclusive scan of hist[0, nbins): thread t owns bins 2t, 2t+1
    const uint32_t b0 = 2 * tid;
    const uint32_t h0 = b0 < pb.geo.nbins ? s.hist[b0] : 0u;
    const uint32_t h1 = b0 + 1 < pb.geo.nbins ? s.hist[b0 + 1] : 0u;
    uint32_t x = h0 + h1;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xFFFFFFFFu, x, o);
        if (lane >= o) x += y;
    }
    if (lane == 31) s.wsum[warp] = x;
    __syncthreads();
    uint32_t before = 0, total = 0;
#pragma unroll
    for (int w = 0; w < kPbWarps; ++w) {
        const uint32_t v = s.wsum[w];
        before += w < warp ? v : 0u;
        total += v;
    }
    const uint32_t e0 = before + x - h0 - h1;
    if (b0 < pb.geo.nbins) {
        s.start[b0] = e0;
        s.gpos[b0] = h0 ? __ldg(pb.boff + b0) + atomicAdd(pb.cur + b0, h0) : 0u;
        s.hist[b0] = 0u;
    }
    if (b0 + 1 < pb.geo.nbins) {
        s.start[b0 + 1] = e0 + h0;
        s.gpos[b0 + 1] = h1 ? __ldg(pb.boff + b0 + 1) + atomicAdd(pb.cur + b0 + 1, h1) : 0u;
        s.hist[b0 + 1] = 0u;
    }
    __syncthreads();                                   // start / gpos of every bin written
#pragma unroll
    for (int k = 0; k < E; ++k) {
        const uint32_t r = (rk[k >> 1] >> ((k & 1) * 16)) & 0xFFFFu;
        if (r == 0xFFFFu) continue;
        const uint32_t b = pb_bin(pb.geo, dst[k]), pos = s.start[b] + r;
        s.stage[pos] = make_uint2(dst[k], __float_as_uint(c[k]));
        s.sbin[pos] = (uint16_t)b;
    }
    __syncthreads();
    for (uint32_t i = tid; i < total; i += kPbThreads) {
        const uint32_t b = s.sbin[i];
        st_stream_v2(pb.pairs + (s.gpos[b] + (i - s.start[b])), s.stage[i]);
    }
}

// Phase 1.  Same page walk as pr_scatter_kernel (tiles of T slots, 16-byte
// evict_first record loads, owner search per 16 bytes), but rounds are
// CTA-uniform so the staging barriers line up.  kCount: only count pairs per
// bin (sizes the bins once per graph).
template <bool kWeighted, bool kCount>
__global__ void __launch_bounds__(kPbThreads, kPbBlocks)
pr_bin_kernel(PageSet ps, const float* __restrict__ x, float* acc, float d, double* dang_out, uint32_t* work_ctr,
              const PbParams pb) {
    constexpr int T = kPbThreads;
    constexpr int E = kPbUnroll * 4;
    __shared__ PrSmem<T> sm;
    extern __shared__ uint4 dyn_smem[];
    float* hacc = reinterpret_cast<float*>(dyn_smem);
    PbSmem& s = *reinterpret_cast<PbSmem*>(hacc + kPbHot);
    const int tid = threadIdx.x;
    if (!kCount)
        for (uint32_t i = tid; i < pb.geo.hot; i += T) hacc[i] = 0.f;
    for (uint32_t i = tid; i < kPbMaxBins; i += T) s.hist[i] = 0u;
    __syncthreads();
    const uint64_t pol = policy_evict_first();
    const uint32_t count = ps.count;
    const uint32_t enc = ps.entry_encoding;
    constexpr uint32_t wshift = kWeighted ? 1 : 0;
    double dang = 0.0;
    HotRun hr{0xFFFFFFFFu, 0.f};
    uint32_t dst[E];
    float cv[E];
    for (;;) {
        if (tid == 0) sm.item = atomicAdd(work_ctr, 1u);
        __syncthreads();
        const uint32_t it = sm.item;
        __syncthreads();
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
            const float c = kCount ? 0.f : d * __ldg(x + vid) / (float)total;
            const uint32_t wend = 1 + len, qend = (wend + 3) >> 2;
            for (uint32_t qb0 = 0; qb0 < qend; qb0 += T * kPbUnroll) {
                uint4 v[kPbUnroll];
#pragma unroll
                for (int u = 0; u < (int)kPbUnroll; ++u) {
                    const uint32_t q = qb0 + tid + u * T;
                    if (q < qend) v[u] = ld_stream_v4(q4 + q, pol);
                }
#pragma unroll
                for (int u = 0; u < (int)kPbUnroll; ++u) {
                    const uint32_t q = qb0 + tid + u * T;
#pragma unroll
                    for (int k = 0; k < 4; ++k) {
                        const uint32_t w = 4 * q + k;
                        const bool e = q < qend && w >= 1 && w < wend;
                        dst[u * 4 + k] = e ? pr_decode(word_of(v[u], k), enc, ps.rvt_start) : kNoEdge;
                        cv[u * 4 + k] = c;
                    }
                }
                pb_round<kCount>(pb, hacc, hr, s, dst, cv);
            }
        } else {
            const uint32_t start = ld32(end - kSpFooter - kSlotBytes);
            for (uint32_t t0 = 0; t0 < nslots; t0 += T) {
                const uint32_t nv = min((uint32_t)T, nslots - t0);
                if ((uint32_t)tid < nv) {
                    const uint8_t* slot = end - kSpFooter - kSlotBytes * (uint64_t)(t0 + tid + 1);
                    sm.off[tid] = ld_stream_u32(slot + 4, pol) >> 2;
                    if ((uint32_t)tid == nv - 1) {
                        if (t0 + nv < nslots) {
                            sm.off[nv] = ld_stream_u32(slot - kSlotBytes + 4, pol) >> 2;
                        } else {
                            const uint32_t o = ld_stream_u32(slot + 4, pol);
                            sm.off[nv] = (o >> 2) + 1 + (ld32(data + o) << wshift);
                        }
                    }
                }
                __syncthreads();
                if (!kCount && (uint32_t)tid < nv) {
                    const uint32_t deg = (sm.off[tid + 1] - sm.off[tid] - 1) >> wshift;
                    const float xv = ld_stream_f32(x + start + t0 + tid, pol);
                    float c = 0.f;
                    if (deg == 0) dang += (double)xv;     // dangling mass (R3)
                    else c = d * xv / (float)deg;
                    sm.c[tid] = c;
                }
                __syncthreads();
                const uint32_t W0 = sm.off[0], W1 = sm.off[nv];
                const uint32_t qbeg = W0 >> 2, qend = (W1 + 3) >> 2;
                for (uint32_t qb0 = qbeg; qb0 < qend; qb0 += T * kPbUnroll) {
                    uint4 v[kPbUnroll];
#pragma unroll
                    for (int u = 0; u < (int)kPbUnroll; ++u) {
                        const uint32_t q = qb0 + tid + u * T;
                        if (q < qend) v[u] = ld_stream_v4(q4 + q, pol);
                    }
#pragma unroll
                    for (int u = 0; u < (int)kPbUnroll; ++u) {
                        const uint32_t q = qb0 + tid + u * T;
#pragma unroll
                        for (int k = 0; k < 4; ++k) dst[u * 4 + k] = kNoEdge;
                        if (q >= qend) continue;
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
                            const uint32_t rel = w - cur;     // 0 = ADJLIST_SZ word; > deg = weight words
                            if (rel == 0 || rel > ((nxt - cur - 1) >> wshift)) continue;
                            dst[u * 4 + k] = pr_decode(word_of(v[u], k), enc, ps.rvt_start);
                            cv[u * 4 + k] = kCount ? 0.f : sm.c[j];
                        }
                    }
                    pb_round<kCount>(pb, hacc, hr, s, dst, cv);
                }
                __syncthreads();
            }
        }
    }
    __syncthreads();
    if (kCount) {
        for (uint32_t b = tid; b < pb.geo.nbins; b += T)
            if (s.hist[b]) atomicAdd(pb.count + b, (unsigned long long)s.hist[b]);
        return;
    }
    hr.flush(hacc);
    __syncthreads();
    for (uint32_t i = tid; i < pb.geo.hot; i += T) {
        const float v = hacc[i];
        if (v != 0.f) atomicAdd(acc + i, v);
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) dang += __shfl_down_sync(0xFFFFFFFFu, dang, o);
    if ((tid & 31) == 0 && dang != 0.0) atomicAdd(dang_out, dang);
}

__device__ __forceinline__ uint2 ld_stream_pair(const uint2* p, uint64_t pol) { return ld_stream_v2(p, pol); }

__device__ __forceinline__ void red_v4(float* p, float4 v) {
    asm volatile("red.global.add.v4.f32 [%0], {%1,%2,%3,%4};" ::"l"(p), "f"(v.x), "f"(v.y), "f"(v.z), "f"(v.w)
                 : "memory");
}

// Phase 2.  items[i] = (bin, first pair, end pair) relative to the bin start;
// the bin's filled length cur[b] clips the end.
template <int T>
__global__ void __launch_bounds__(T, 1)
pr_apply_kernel(const PbParams pb, const uint4* __restrict__ items, uint32_t n_items, uint32_t* work_ctr, float* acc) {
    extern __shared__ uint4 dyn_smem[];
    float* sacc = reinterpret_cast<float*>(dyn_smem);
    __shared__ uint32_t s_item;
    const int tid = threadIdx.x;
    const uint64_t pol = policy_evict_first();
    const uint32_t bw = 1u << pb.geo.fine_shift;
    constexpr int U = 4;
    for (;;) {
        if (tid == 0) s_item = atomicAdd(work_ctr, 1u);
        __syncthreads();
        const uint32_t it = s_item;
        __syncthreads();
        if (it >= n_items) break;
        const uint4 item = __ldg(items + it);
        const uint32_t b = item.x;
        const uint32_t filled = __ldg(pb.cur + b);
        const uint32_t lo = item.y, hi = min(item.z, filled);
        if (lo >= hi) continue;                                // CTA-uniform
        const uint2* pr = pb.pairs + __ldg(pb.boff + b);
        if (b < pb.geo.nfine) {
            const uint32_t base = pb.geo.hot + (b << pb.geo.fine_shift);
            for (uint32_t i = tid; i < bw; i += T) sacc[i] = 0.f;
            __syncthreads();
            for (uint32_t i0 = lo + tid; i0 < hi; i0 += T * U) {
                uint2 e[U];
#pragma unroll
                for (int u = 0; u < U; ++u)
                    if (i0 + u * T < hi) e[u] = ld_stream_pair(pr + i0 + u * T, pol);
#pragma unroll
                for (int u = 0; u < U; ++u)
                    if (i0 + u * T < hi) atomicAdd(sacc + (e[u].x - base), __uint_as_float(e[u].y));
            }
            __syncthreads();
            const float4* s4 = reinterpret_cast<const float4*>(sacc);
            for (uint32_t j = tid; j < bw / 4; j += T) {
                const float4 v = s4[j];
                if (v.x == 0.f && v.y == 0.f && v.z == 0.f && v.w == 0.f) continue;
                const uint64_t g = (uint64_t)base + 4 * j;
                if (g + 4 <= pb.geo.n) {
                    red_v4(acc + g, v);
                } else {
                    const float a[4] = {v.x, v.y, v.z, v.w};
                    for (int k = 0; k < 4; ++k)
                        if (g + k < pb.geo.n && a[k] != 0.f) atomicAdd(acc + g + k, a[k]);
                }
            }
            __syncthreads();                                   // sacc is zeroed by the next item
        } else {
            for (uint32_t i0 = lo + tid; i0 < hi; i0 += T * U) {
                uint2 e[U];
#pragma unroll
                for (int u = 0; u < U; ++u)
                    if (i0 + u * T < hi) e[u] = ld_stream_pair(pr + i0 + u * T, pol);
#pragma unroll
                for (int u = 0; u < U; ++u)
                    if (i0 + u * T < hi) atomicAdd(acc + e[u].x, __uint_as_float(e[u].y));
            }
        }
    }
}

enum { kBufX = 20, kBufAcc, kBufDang, kBufPrCtr, kBufRouteSend, kBufRouteRecv, kBufRouteHot, kBufRouteHotIn,
       kBufRouteCnt, kBufRouteList, kBufPbPairs = 90, kBufPbMeta, kBufPbItems, kBufPbCount };

inline size_t pb_bin_smem() { return (size_t)kPbHot * 4 + sizeof(PbSmem); }

inline uint32_t env_u32(const char* name, uint32_t dflt) {
    const char* v = getenv(name);
    return v ? (uint32_t)atol(v) : dflt;
}

// Bin geometry, pair counts (once per graph and geometry, one counting sweep
// over this rank's resident pages), bin offsets and phase-2 work items.
// *ok = false when the pairs do not fit the u32 offsets (caller keeps the
// plain scatter).
int pb_plan(Context* c, const Graph* g, cudaStream_t s, PbParams& pb, uint4** d_items, uint32_t* n_items, bool* ok) {
    const uint64_t n = g->n;
    PbGeom& geo = pb.geo;
    uint32_t hot = std::min<uint32_t>(env_u32("GTS_PB_HOT", kPbHot), kPbHot) & ~3u;
    if ((uint64_t)hot > n) hot = (uint32_t)((n + 3) & ~3ull);
    geo.hot = hot;
    geo.fine_shift = std::max<uint32_t>(2, std::min<uint32_t>(env_u32("GTS_PB_FINE_SHIFT", kPbFineShiftMax), kPbFineShiftMax));
    const uint64_t rest = n > hot ? n - hot : 0;
    const uint64_t bw = 1ull << geo.fine_shift;
    geo.nfine = (uint32_t)std::min<uint64_t>((rest + bw - 1) / bw, std::min<uint32_t>(env_u32("GTS_PB_NFINE", 512), kPbMaxBins / 2));
    geo.fine_end = hot + ((uint64_t)geo.nfine << geo.fine_shift);
    const uint64_t rest2 = n > geo.fine_end ? n - geo.fine_end : 0;
    uint32_t cs = env_u32("GTS_PB_COARSE_SHIFT", 21);
    while (cs < 40 && (rest2 >> cs) + 1 > kPbMaxBins - geo.nfine) ++cs;
    geo.coarse_shift = cs;
    const uint32_t ncoarse = (uint32_t)((rest2 + (1ull << cs) - 1) >> cs);
    geo.nbins = geo.nfine + ncoarse;
    geo.n = n;
    DevGraph& dg = c->dg;
    const uint64_t key = (g->uid << 24) ^ ((uint64_t)hot << 8) ^ ((uint64_t)geo.fine_shift << 40) ^
                         ((uint64_t)geo.nfine << 44) ^ ((uint64_t)cs << 56) ^ 1;
    uint32_t* meta;   // boff[kPbMaxBins] | cur[kPbMaxBins]
    GTS_TRY(c->buf(kBufPbMeta, 2 * kPbMaxBins * 4, (void**)&meta));
    pb.boff = meta;
    pb.cur = meta + kPbMaxBins;
    PageSet ps;
    ps.base = dg.pages;
    ps.list = dg.all_local ? nullptr : dg.local_list;
    ps.loc = dg.loc;
    ps.d_count = nullptr;
    ps.count = dg.n_local;
    ps.page_bytes = g->page_bytes;
    ps.mode = dg.all_local ? kAddrByPid : kAddrByLoc;
    ps.entry_encoding = g->entry_encoding;
    ps.rvt_start = dg.rvt_start;
    const size_t smem = pb_bin_smem();
    static bool attr = false;
    if (!attr) {
        for (const void* k : {(const void*)pr_bin_kernel<false, false>, (const void*)pr_bin_kernel<true, false>,
                              (const void*)pr_bin_kernel<false, true>, (const void*)pr_bin_kernel<true, true>})
            GTS_CUDA(cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
        GTS_CUDA(cudaFuncSetAttribute((const void*)pr_apply_kernel<1024>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                      4 << kPbFineShiftMax));
        attr = true;
    }
    if (dg.pb_key != key) {
        unsigned long long* cnt;
        uint32_t* ctr;
        GTS_TRY(c->buf(kBufPbCount, kPbMaxBins * 8 + 8, (void**)&cnt));
        ctr = reinterpret_cast<uint32_t*>(cnt + kPbMaxBins);
        GTS_CUDA(cudaMemsetAsync(cnt, 0, kPbMaxBins * 8 + 8, s));
        PbParams pc = pb;
        pc.count = cnt;
        const float dz = 0.f;
        const float* xz = nullptr;
        float* az = nullptr;
        double* dd = nullptr;
        const void* kc = g->weighted ? (const void*)pr_bin_kernel<true, true> : (const void*)pr_bin_kernel<false, true>;
        void* a[] = {(void*)&ps, (void*)&xz, (void*)&az, (void*)&dz, (void*)&dd, (void*)&ctr, (void*)&pc};
        GTS_CUDA(cudaLaunchKernel(kc, dim3(c->num_sms * kPbBlocks), dim3(kPbThreads), a, smem, s));
        GTS_CUDA(cudaGetLastError());
        dg.pb_count.assign(kPbMaxBins, 0);
        GTS_CUDA(cudaMemcpyAsync(dg.pb_count.data(), cnt, kPbMaxBins * 8, cudaMemcpyDeviceToHost, s));
        GTS_CUDA(cudaStreamSynchronize(s));
        dg.pb_key = key;
    }
    std::vector<uint32_t> boff(kPbMaxBins, 0);
    uint64_t tot = 0;
    for (uint32_t b = 0; b < geo.nbins; ++b) {
        boff[b] = (uint32_t)tot;
        tot += dg.pb_count[b];
        if (tot >= (1ull << 32)) {
            *ok = false;
            return GTS_OK;
        }
    }
    const uint32_t chunk = std::max<uint32_t>(1024, env_u32("GTS_PB_CHUNK", 1u << 17));
    std::vector<uint4> items;
    for (uint32_t b = 0; b < geo.nbins; ++b)
        for (uint64_t lo = 0; lo < dg.pb_count[b]; lo += chunk)
            items.push_back(make_uint4(b, (uint32_t)lo, (uint32_t)std::min<uint64_t>(lo + chunk, dg.pb_count[b]), 0));
    GTS_TRY(c->buf(kBufPbPairs, std::max<uint64_t>(tot, 1) * 8, (void**)&pb.pairs));
    GTS_TRY(c->buf(kBufPbItems, std::max<size_t>(items.size(), 1) * sizeof(uint4), (void**)d_items));
    GTS_CUDA(cudaMemcpyAsync(meta, boff.data(), kPbMaxBins * 4, cudaMemcpyHostToDevice, s));
    if (!items.empty())
        GTS_CUDA(cudaMemcpyAsync(*d_items, items.data(), items.size() * sizeof(uint4), cudaMemcpyHostToDevice, s));
    GTS_CUDA(cudaStreamSynchronize(s));        // host vectors go out of scope
    *n_items = (uint32_t)items.size();
    *ok = true;
    return GTS_OK;
}

}  // namespace gts

using namespace gts;

extern "C" int gts_pagerank(gts_context* c, const gts_graph* g, uint32_t iters, double damping, uint32_t dangling,
                            const gts_run_config* cfg, float* rank_out, gts_run_stats* st) {
    clear_error();
    const double t_start = now_s();
    gts_run_config rc;
    GTS_TRY(validate_common(c, g, cfg, &rc));
    if (!rank_out) return fail(GTS_EINVAL, "NULL output");
    if (!(damping >= 0.0 && damping <= 1.0)) return fail(GTS_EINVAL, "damping must be in [0,1]");
    if (dangling > GTS_DANGLING_DROP) return fail(GTS_EINVAL, "unknown dangling mode %u", dangling);
    const uint64_t n = g->n;
    const bool streamed = choose_streamed(c, g, rc, 8 * n);
    // Strategy-S with routed updates: N > 1 ranks, or (tests, one GPU) GTS_VIRTUAL_RANKS=V
    // virtual ranks run one after another on this GPU with an in-memory exchange
    const char* vre = getenv("GTS_VIRTUAL_RANKS");
    const int vranks = (rc.strategy != GTS_STRATEGY_P && c->world == 1 && vre) ? std::max(1, atoi(vre)) : 1;
    const bool virt = vranks > 1;
    const bool bcast = rc.strategy == GTS_STRATEGY_S_BCAST;
    const bool route = (rc.strategy == GTS_STRATEGY_S || bcast) && (c->world > 1 || virt);
    const int R = virt ? vranks : c->world;
    if (route && R > kMaxRanks) return fail(GTS_EUNSUPPORTED, "Strategy-S routing supports at most %d ranks", kMaxRanks);
    double upload_s = 0;
    GTS_TRY(ensure_graph(c, g, rc.strategy, !streamed, &upload_s));
    const bool timing = rc.flags & GTS_RUN_TIMING;
    float *x, *acc;
    double* dang;
    uint32_t* ctr;
    GTS_TRY(c->buf(kBufX, n * 4, (void**)&x));
    GTS_TRY(c->buf(kBufAcc, n * 4, (void**)&acc));
    GTS_TRY(c->buf(kBufDang, 2 * sizeof(double), (void**)&dang));
    GTS_TRY(c->buf(kBufPrCtr, 4, (void**)&ctr));
    cudaStream_t s = c->stream;
    // scatter variant: degree-ordered graphs use the dense hot set held by one 1024-thread CTA per
    // SM (53,248 floats; GTS_PR_BIG=0 selects two 512-thread CTAs with 24,576 each, 3% slower
    // on RMAT-27); natural-order graphs the hash table; routed Strategy-S always the dense set
    const uint32_t micro = (rc.flags & GTS_MICRO_MASK) >> 8;
    if (micro > (GTS_MICRO_TILE >> 8)) return fail(GTS_EINVAL, "unknown GTS_MICRO value");
    if (micro && route) return fail(GTS_EUNSUPPORTED, "GTS_MICRO_* techniques run without Strategy-S routing");
    const char* pbig = getenv("GTS_PR_BIG");
    const bool big = (g->ordered || route) && (!pbig || atoi(pbig) > 0);
    const int mode = route ? kRoute : (g->ordered ? kDense : kHash);
    // warp-window page walk (record-start masks instead of a binary search per 16 bytes)
    // (measured on RMAT-27: 12.48 vs 12.24 ms for the tile walk, so opt-in: GTS_PR_WW=1)
    const char* wwe = getenv("GTS_PR_WW");
    const bool ww = mode == kDense && big && wwe && atoi(wwe) > 0;
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
    } else if (mode == kHash) {
        kern = g->weighted ? (const void*)pr_scatter_kernel<true, kHash, kThreads, 2, 0>
                           : (const void*)pr_scatter_kernel<false, kHash, kThreads, 2, 0>;
        dyn = pr_dyn_smem<kHash, 0>();
        threads = kThreads;
        n_hot = 0;
    } else if (mode == kRoute) {
        kern = g->weighted ? (const void*)pr_scatter_kernel<true, kRoute, 1024, 1, kHotDenseBig>
                           : (const void*)pr_scatter_kernel<false, kRoute, 1024, 1, kHotDenseBig>;
        dyn = pr_dyn_smem<kRoute, kHotDenseBig>();
        threads = 1024;
        n_hot = (uint32_t)std::min<uint64_t>(n, kHotDenseBig);
    } else if (!big) {
        kern = g->weighted ? (const void*)pr_scatter_kernel<true, kDense, kThreads, 2, kHotDense>
                           : (const void*)pr_scatter_kernel<false, kDense, kThreads, 2, kHotDense>;
        dyn = pr_dyn_smem<kDense, kHotDense>();
        threads = kThreads;
        n_hot = (uint32_t)std::min<uint64_t>(n, kHotDense);
    } else if (ww) {
        kern = g->weighted ? (const void*)pr_scatter_ww_kernel<true, 1024, 1, kHotDenseBig>
                           : (const void*)pr_scatter_ww_kernel<false, 1024, 1, kHotDenseBig>;
        dyn = pr_dyn_smem<kDense, kHotDenseBig>();
        threads = 1024;
        n_hot = (uint32_t)std::min<uint64_t>(n, kHotDenseBig);
    } else {
        kern = g->weighted ? (const void*)pr_scatter_kernel<true, kDense, 1024, 1, kHotDenseBig>
                           : (const void*)pr_scatter_kernel<false, kDense, 1024, 1, kHotDenseBig>;
        dyn = pr_dyn_smem<kDense, kHotDenseBig>();
        threads = 1024;
        n_hot = (uint32_t)std::min<uint64_t>(n, kHotDenseBig);
    }
    GTS_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)dyn));
    int grid = 0;
    GTS_TRY(sms_grid(c, kern, threads, dyn, &grid));
    // L2 persistence for the hot head of WA: on a degree-ordered graph the most
    // updated entries are acc[0, W) (W = 96 MiB by default, clipped to the
    // device's persisting-L2 limit); GTS_L2_PERSIST=<MiB> overrides, 0 disables.
    bool persist = false;
    const char* pe = getenv("GTS_L2_PERSIST");
    const char* pbe = getenv("GTS_PR_BINNED");
    bool binned = g->ordered && !streamed && !route && !micro && pbe && atoi(pbe) > 0;
    if (g->ordered && !route && !binned && (!pe || atol(pe) > 0)) {
        const size_t want = std::min<size_t>((size_t)(pe ? atol(pe) : 96) << 20, n * 4);
        if (want > 0) {
            GTS_TRY(persist_window(c, s, acc, want));
            persist = true;
        }
    }
    const int eg = c->num_sms * 4;
    pr_init_kernel<<<eg, 256, 0, s>>>(x, acc, n, (float)(1.0 / (double)n));
    GTS_CUDA(cudaMemsetAsync(dang, 0, 2 * sizeof(double), s));
    uint64_t launches = 1, main_launches = 0, nccl_bytes = 0;
    SweepStats ss;
    float dmp = (float)damping;
    const uint32_t* hk = c->dg.hot_keys;
    const char* hde = getenv("GTS_HYBRID_DEG");
    const uint32_t hybrid_deg = hde ? (uint32_t)std::max(1L, atol(hde)) : 8u;
    auto scatter = [&](const PageSet& ps, int cap, double* D, const RouteParams& rp) -> int {
        GTS_CUDA(cudaMemsetAsync(ctr, 0, 4, s));
        std::pair<cudaEvent_t, cudaEvent_t> e2;
        if (timing) { e2 = c->t_main.next(); cudaEventRecord(e2.first, s); }
        PageSet p2 = ps;
        p2.hybrid_deg = hybrid_deg;
        void* args_full[] = {(void*)&p2, (void*)&x, (void*)&acc, (void*)&hk, (void*)&dmp, (void*)&D,
                             (void*)&ctr, (void*)&n_hot, (void*)&rp};
        void* args_ww[] = {(void*)&p2, (void*)&x, (void*)&acc, (void*)&dmp, (void*)&D, (void*)&ctr, (void*)&n_hot};
        void** args = ww && !micro ? args_ww : args_full;
        cudaLaunchConfig_t lc;
        std::memset(&lc, 0, sizeof(lc));
        lc.gridDim = dim3(std::min(grid, cap));
        lc.blockDim = dim3(threads);
        lc.dynamicSmemBytes = dyn;
        lc.stream = s;
        GTS_CUDA(cudaLaunchKernelExC(&lc, kern, args));
        if (timing) cudaEventRecord(e2.second, s);
        GTS_CUDA(cudaGetLastError());
        ++main_launches;
        return GTS_OK;
    };
    RouteParams rp0;
    std::memset(&rp0, 0, sizeof(rp0));
    // binned scatter (section 6b of DESIGN.md): degree-ordered, resident, not routed
    PbParams pb;
    std::memset(&pb, 0, sizeof(pb));
    uint4* d_items = nullptr;
    uint32_t n_items = 0;
    if (binned) {
        GTS_TRY(pb_plan(c, g, s, pb, &d_items, &n_items, &binned));
        if (binned) GTS_TRY(c->buf(kBufPrCtr, 8, (void**)&ctr));
    }
    auto binned_scatter = [&](const PageSet& ps, double* D) -> int {
        GTS_CUDA(cudaMemsetAsync(ctr, 0, 8, s));
        GTS_CUDA(cudaMemsetAsync(pb.cur, 0, (size_t)pb.geo.nbins * 4, s));
        std::pair<cudaEvent_t, cudaEvent_t> e2;
        if (timing) { e2 = c->t_main.next(); cudaEventRecord(e2.first, s); }
        const void* k1 = g->weighted ? (const void*)pr_bin_kernel<true, false> : (const void*)pr_bin_kernel<false, false>;
        void* a1[] = {(void*)&ps, (void*)&x, (void*)&acc, (void*)&dmp, (void*)&D, (void*)&ctr, (void*)&pb};
        GTS_CUDA(cudaLaunchKernel(k1, dim3(c->num_sms * kPbBlocks), dim3(kPbThreads), a1, pb_bin_smem(), s));
        uint32_t* ctr2 = ctr + 1;
        void* a2[] = {(void*)&pb, (void*)&d_items, (void*)&n_items, (void*)&ctr2, (void*)&acc};
        GTS_CUDA(cudaLaunchKernel((const void*)pr_apply_kernel<1024>, dim3(c->num_sms), dim3(1024), a2,
                                  (size_t)4 << pb.geo.fine_shift, s));
        if (timing) cudaEventRecord(e2.second, s);
        GTS_CUDA(cudaGetLastError());
        ++main_launches;
        ++launches;
        return GTS_OK;
    };
    if (!route) {
        const uint32_t* d_list = (c->dg.all_local && !streamed) ? nullptr : c->dg.local_list;
        for (uint32_t it = 0; it < iters; ++it) {
            double* D = dang + (it & 1);
            std::pair<cudaEvent_t, cudaEvent_t> ev;
            GTS_TRY(sweep_pages(c, g, rc, streamed, &c->dg.h_local_list, d_list, c->dg.n_local, nullptr,
                                [&](const PageSet& ps, int cap) -> int {
                                    return binned ? binned_scatter(ps, D) : scatter(ps, cap, D, rp0);
                                }, &ss));
            if (c->world > 1) {         // Strategy-P: every replica receives the full sum
                if (timing) { ev = c->t_merge.next(); cudaEventRecord(ev.first, s); }
                GTS_NCCL(ncclGroupStart());
                GTS_NCCL(ncclAllReduce(acc, acc, n, ncclFloat32, ncclSum, c->comm, s));
                GTS_NCCL(ncclAllReduce(D, D, 1, ncclFloat64, ncclSum, c->comm, s));
                GTS_NCCL(ncclGroupEnd());
                if (timing) cudaEventRecord(ev.second, s);
                nccl_bytes += n * 4 + 8;
            }
            if (timing) { ev = c->t_finish.next(); cudaEventRecord(ev.first, s); }
            pr_finish_kernel<<<2 * eg, 256, 0, s>>>(x, acc, n, 0, n, damping, D, dang + ((it + 1) & 1),
                                                 dangling == GTS_DANGLING_UNIFORM ? 1 : 0, 0);
            if (timing) cudaEventRecord(ev.second, s);
            ++launches;
        }
    } else {
        // ---- Strategy-S, routed: rank r owns WA [vr[r], vr[r+1]) and the pages whose sources lie in it
        std::vector<int32_t> owner;
        std::vector<uint64_t> vr;
        partition(g, GTS_STRATEGY_S, R, owner, vr);
        std::vector<std::vector<uint32_t>> plist(R);          // pages of each (virtual) rank
        for (uint64_t j = 0; j < g->num_pages; ++j)
            for (int r = 0; r < R; ++r)
                if (bcast || owner[j] == r) plist[r].push_back((uint32_t)j);   // S_BCAST: every rank, every page
        const int me = virt ? -1 : c->rank;
        const int r0 = virt ? 0 : me, r1 = virt ? R : me + 1;  // ranks simulated by this process
        std::vector<uint32_t> pl_off(R + 1, 0);
        for (int r = 0; r < R; ++r) pl_off[r + 1] = pl_off[r] + (uint32_t)plist[r].size();
        uint32_t* d_plist = nullptr;              // (S_BCAST: every rank lists every page)
        GTS_TRY(c->buf(kBufRouteList, std::max<uint64_t>(pl_off[R], 1) * 4, (void**)&d_plist));
        {
            std::vector<uint32_t> flat;
            for (int r = 0; r < R; ++r) flat.insert(flat.end(), plist[r].begin(), plist[r].end());
            GTS_CUDA(cudaMemcpyAsync(d_plist, flat.data(), flat.size() * 4, cudaMemcpyHostToDevice, s));
            GTS_CUDA(cudaStreamSynchronize(s));
        }
        auto make_rp = [&](int r) {
            RouteParams rp;
            std::memset(&rp, 0, sizeof(rp));
            for (int k = 0; k <= R; ++k) rp.vr[k] = vr[k];
            rp.lo = vr[r];
            rp.hi = vr[r + 1];
            rp.nranks = R;
            rp.acc_loc = acc + vr[r];
            rp.drop_remote = bcast ? 1 : 0;
            return rp;
        };
        auto pages_of = [&](int r, const uint32_t*& d, uint32_t& cnt) {
            d = d_plist + pl_off[r];
            cnt = pl_off[r + 1] - pl_off[r];
        };
        // send capacities: remote cold edges per (sender, owner), counted once per call
        unsigned long long* d_cnt64;
        // u64 capacities [kMaxRanks^2] | u32 flags[8] | send counts [kMaxRanks^2] | recv counts [kMaxRanks]
        GTS_TRY(c->buf(kBufRouteCnt, sizeof(unsigned long long) * kMaxRanks * kMaxRanks +
                                         (8 + kMaxRanks * kMaxRanks + kMaxRanks) * 4, (void**)&d_cnt64));
        GTS_CUDA(cudaMemsetAsync(d_cnt64, 0, sizeof(unsigned long long) * kMaxRanks * kMaxRanks, s));
        const void* kcount = g->weighted ? (const void*)route_count_kernel<true> : (const void*)route_count_kernel<false>;
        int cgrid = 0;
        GTS_TRY(sms_grid(c, kcount, kThreads, 0, &cgrid));
        for (int r = r0; r < r1 && !bcast; ++r) {
            RouteParams rp = make_rp(r);
            const uint32_t* dl;
            uint32_t cnt;
            pages_of(r, dl, cnt);
            std::vector<uint32_t> hl(plist[r]);
            GTS_TRY(sweep_pages(c, g, rc, streamed, &hl, dl, cnt, nullptr, [&](const PageSet& ps, int cap) -> int {
                GTS_CUDA(cudaMemsetAsync(ctr, 0, 4, s));
                unsigned long long* out = d_cnt64 + (size_t)r * kMaxRanks;
                void* args[] = {(void*)&ps, (void*)&rp, (void*)&n_hot, (void*)&out, (void*)&ctr};
                GTS_CUDA(cudaLaunchKernel(kcount, dim3(std::min(cgrid, cap)), dim3(kThreads), args, 0, s));
                ++launches;
                return GTS_OK;
            }, &ss));
        }
        std::vector<unsigned long long> cap64((size_t)kMaxRanks * kMaxRanks, 0);
        GTS_CUDA(cudaMemcpyAsync(cap64.data(), d_cnt64, cap64.size() * 8, cudaMemcpyDeviceToHost, s));
        GTS_CUDA(cudaStreamSynchronize(s));
        uint32_t* d_flags = reinterpret_cast<uint32_t*>(d_cnt64 + (size_t)kMaxRanks * kMaxRanks);  // [0] overflow
        uint32_t* d_scnt = d_flags + 8;            // send counts [R] per simulated rank (R x R in virtual mode)
        uint32_t* d_rcnt = d_flags + 8 + kMaxRanks * kMaxRanks;
        if (!virt && !bcast) {   // everyone learns what it will receive: all-gather the capacity rows
            uint32_t* d_caprow;
            uint32_t* d_capall;
            GTS_TRY(c->buf(kBufRouteHotIn + 10, (size_t)(R + R * R) * 4, (void**)&d_caprow));
            d_capall = d_caprow + R;
            std::vector<uint32_t> row(R);
            for (int p = 0; p < R; ++p) row[p] = (uint32_t)cap64[(size_t)me * kMaxRanks + p];
            GTS_CUDA(cudaMemcpyAsync(d_caprow, row.data(), R * 4, cudaMemcpyHostToDevice, s));
            GTS_NCCL(ncclAllGather(d_caprow, d_capall, R, ncclUint32, c->comm, s));
            std::vector<uint32_t> all((size_t)R * R);
            GTS_CUDA(cudaMemcpyAsync(all.data(), d_capall, all.size() * 4, cudaMemcpyDeviceToHost, s));
            GTS_CUDA(cudaStreamSynchronize(s));
            for (int a = 0; a < R; ++a)
                for (int p = 0; p < R; ++p) cap64[(size_t)a * kMaxRanks + p] = all[(size_t)a * R + p];
        }
        // buffers: send regions of each simulated rank; receive regions (real ranks)
        std::vector<uint32_t> soff((size_t)R * kMaxRanks, 0), roff(kMaxRanks, 0);
        uint64_t stot = 0, rtot = 0;
        for (int r = r0; r < r1; ++r)
            for (int p = 0; p < R; ++p) {
                soff[(size_t)r * kMaxRanks + p] = (uint32_t)stot;
                stot += cap64[(size_t)r * kMaxRanks + p];
            }
        if (!virt)
            for (int p = 0; p < R; ++p) {
                roff[p] = (uint32_t)rtot;
                rtot += cap64[(size_t)p * kMaxRanks + me];
            }
        if (stot >= (1ull << 32) || rtot >= (1ull << 32)) return fail(GTS_EOVERFLOW, "route buffers exceed 2^32 pairs");
        uint2 *d_send, *d_recv = nullptr;
        float *d_hot, *d_hot_in = nullptr;
        GTS_TRY(c->buf(kBufRouteSend, std::max<uint64_t>(stot, 1) * 8, (void**)&d_send));
        if (!virt) GTS_TRY(c->buf(kBufRouteRecv, std::max<uint64_t>(rtot, 1) * 8, (void**)&d_recv));
        GTS_TRY(c->buf(kBufRouteHot, (size_t)(r1 - r0) * std::max<uint32_t>(n_hot, 1) * 4, (void**)&d_hot));
        if (!virt) GTS_TRY(c->buf(kBufRouteHotIn, std::max<uint32_t>(n_hot, 1) * 4, (void**)&d_hot_in));
        GTS_CUDA(cudaMemsetAsync(d_hot, 0, (size_t)(r1 - r0) * std::max<uint32_t>(n_hot, 1) * 4, s));
        GTS_CUDA(cudaMemsetAsync(d_flags, 0, 4, s));
        uint32_t* d_soff;                          // device copy of the send offsets (for apply)
        GTS_TRY(c->buf(kBufRouteHotIn + 11, (size_t)(R * kMaxRanks + kMaxRanks) * 4, (void**)&d_soff));
        GTS_CUDA(cudaMemcpyAsync(d_soff, soff.data(), soff.size() * 4, cudaMemcpyHostToDevice, s));
        GTS_CUDA(cudaMemcpyAsync(d_soff + R * kMaxRanks, roff.data(), kMaxRanks * 4, cudaMemcpyHostToDevice, s));
        std::vector<uint32_t> h_scnt(kMaxRanks * kMaxRanks), h_rcnt(kMaxRanks);
        for (uint32_t it = 0; it < iters; ++it) {
            double* D = dang + (it & 1);
            std::pair<cudaEvent_t, cudaEvent_t> ev;
            GTS_CUDA(cudaMemsetAsync(d_scnt, 0, (size_t)kMaxRanks * kMaxRanks * 4, s));
            for (int r = r0; r < r1; ++r) {
                RouteParams rp = make_rp(r);
                rp.hot_out = d_hot + (size_t)(r - r0) * n_hot;
                rp.send = d_send;
                rp.send_cnt = d_scnt + (size_t)r * kMaxRanks;
                rp.overflow = d_flags;
                for (int p = 0; p < R; ++p) {
                    rp.send_off[p] = soff[(size_t)r * kMaxRanks + p];
                    rp.send_cap[p] = (uint32_t)cap64[(size_t)r * kMaxRanks + p];
                }
                const uint32_t* dl;
                uint32_t cnt;
                pages_of(r, dl, cnt);
                std::vector<uint32_t> hl(plist[r]);
                GTS_TRY(sweep_pages(c, g, rc, streamed, &hl, dl, cnt, nullptr,
                                    [&](const PageSet& ps, int cap) -> int { return scatter(ps, cap, D, rp); }, &ss));
            }
            if (timing) { ev = c->t_merge.next(); cudaEventRecord(ev.first, s); }
            if (virt) {                // in-memory exchange: every sender's pairs and hot partials land in acc
                for (int r = 0; r < R; ++r) {
                    route_apply_kernel<<<eg, 256, 0, s>>>(d_send, d_soff + (size_t)r * kMaxRanks,
                                                          d_scnt + (size_t)r * kMaxRanks, R, acc, 0);
                    dense_add_kernel<<<eg, 256, 0, s>>>(acc, d_hot + (size_t)r * n_hot, 0, n_hot);
                    launches += 2;
                }
            } else if (bcast) {        // paper-literal S: no exchange, only the dangling mass
                GTS_NCCL(ncclAllReduce(D, D, 1, ncclFloat64, ncclSum, c->comm, s));
                nccl_bytes += 8;
            } else {
                const uint32_t* scnt_me = d_scnt + (size_t)me * kMaxRanks;
                GTS_NCCL(ncclGroupStart());
                for (int p = 0; p < R; ++p) {
                    if (p == me) continue;
                    GTS_NCCL(ncclSend(scnt_me + p, 1, ncclUint32, p, c->comm, s));
                    GTS_NCCL(ncclRecv(d_rcnt + p, 1, ncclUint32, p, c->comm, s));
                }
                for (int q = 0; q < R; ++q) {  // hot partials: reduce each owner's slice of [0, n_hot)
                    const uint64_t a = std::min<uint64_t>(vr[q], n_hot), b = std::min<uint64_t>(vr[q + 1], n_hot);
                    if (b > a)
                        GTS_NCCL(ncclReduce(d_hot + a, d_hot_in + a, b - a, ncclFloat32, ncclSum, q, c->comm, s));
                }
                GTS_NCCL(ncclGroupEnd());
                GTS_CUDA(cudaMemcpyAsync(h_scnt.data(), scnt_me, R * 4, cudaMemcpyDeviceToHost, s));
                GTS_CUDA(cudaMemcpyAsync(h_rcnt.data(), d_rcnt, R * 4, cudaMemcpyDeviceToHost, s));
                GTS_CUDA(cudaStreamSynchronize(s));
                GTS_NCCL(ncclGroupStart());
                for (int p = 0; p < R; ++p) {
                    if (p == me) continue;
                    if (h_scnt[p])
                        GTS_NCCL(ncclSend(d_send + soff[(size_t)me * kMaxRanks + p], (size_t)h_scnt[p] * 2, ncclUint32,
                                          p, c->comm, s));
                    if (h_rcnt[p])
                        GTS_NCCL(ncclRecv(d_recv + roff[p], (size_t)h_rcnt[p] * 2, ncclUint32, p, c->comm, s));
                    nccl_bytes += (uint64_t)h_scnt[p] * 8;
                }
                GTS_NCCL(ncclGroupEnd());
                GTS_CUDA(cudaMemsetAsync(d_rcnt + me, 0, 4, s));
                route_apply_kernel<<<eg, 256, 0, s>>>(d_recv, d_soff + R * kMaxRanks, d_rcnt, R, acc, 0);
                const uint64_t a = std::min<uint64_t>(vr[me], n_hot), b = std::min<uint64_t>(vr[me + 1], n_hot);
                if (b > a) dense_add_kernel<<<eg, 256, 0, s>>>(acc, d_hot_in, a, b);
                GTS_CUDA(cudaMemsetAsync(d_hot, 0, std::max<uint32_t>(n_hot, 1) * 4, s));
                GTS_NCCL(ncclAllReduce(D, D, 1, ncclFloat64, ncclSum, c->comm, s));
                launches += 2;
                nccl_bytes += n_hot * 4 + 8;
            }
            if (timing) { cudaEventRecord(ev.second, s); ev = c->t_finish.next(); cudaEventRecord(ev.first, s); }
            const uint64_t flo = virt ? 0 : vr[me], fhi = virt ? n : vr[me + 1];
            pr_finish_kernel<<<2 * eg, 256, 0, s>>>(x, acc, n, flo, fhi, damping, D, dang + ((it + 1) & 1),
                                                 dangling == GTS_DANGLING_UNIFORM ? 1 : 0, 0);
            if (timing) cudaEventRecord(ev.second, s);
            ++launches;
            if (bcast && !virt && it + 1 < iters) {   // every rank reads every source's RA next iteration
                GTS_NCCL(ncclGroupStart());
                for (int r = 0; r < R; ++r)
                    if (vr[r + 1] > vr[r])
                        GTS_NCCL(ncclBroadcast(x + vr[r], x + vr[r], vr[r + 1] - vr[r], ncclFloat32, r, c->comm, s));
                GTS_NCCL(ncclGroupEnd());
                nccl_bytes += n * 4;
            }
        }
        uint32_t ovf = 0;
        GTS_CUDA(cudaMemcpyAsync(&ovf, d_flags, 4, cudaMemcpyDeviceToHost, s));
        GTS_CUDA(cudaStreamSynchronize(s));
        if (ovf) return fail(GTS_ECUDA, "Strategy-S route buffer overflow (capacity count mismatch)");
        if (!virt) {               // gather every rank's finished range so all ranks return the full vector
            GTS_NCCL(ncclGroupStart());
            for (int r = 0; r < R; ++r)
                if (vr[r + 1] > vr[r])
                    GTS_NCCL(ncclBroadcast(x + vr[r], x + vr[r], vr[r + 1] - vr[r], ncclFloat32, r, c->comm, s));
            GTS_NCCL(ncclGroupEnd());
            nccl_bytes += n * 4;
        }
    }
    launches += main_launches;
    if (persist) {
        GTS_TRY(persist_window(c, s, nullptr, 0));
        // The lines marked persisting stay so until a later call's window (BFS
        // visited, SSSP dist, WCC parents, PageRank acc) replaces them or the
        // context is freed: an explicit cudaCtxResetPersistingL2Cache here
        // measured +20 ms on the following call (GTS_L2_RESET=1 forces it).
        const char* rs = getenv("GTS_L2_RESET");
        if (rs && atoi(rs) != 0) GTS_CUDA(cudaCtxResetPersistingL2Cache());
    }
    GTS_CUDA(cudaGetLastError());
    GTS_TRY(deliver(c, g, reinterpret_cast<const uint32_t*>(x), rank_out, rc.out_location, false));
    if (st) {
        std::memset(st, 0, sizeof(*st));
        st->wall_s = now_s() - t_start;
        st->upload_s = upload_s;
        if (timing) {
            st->main_kernel_s = c->t_main.sum_s();
            st->merge_s = c->t_merge.sum_s();
            st->finish_s = c->t_finish.sum_s();
        }
        st->pages_processed = (uint64_t)c->dg.n_local * iters;
        st->h2d_bytes = ss.h2d_bytes;
        if (timing) st->h2d_s = c->t_h2d.sum_s();
        st->edges_traversed = g->m * (uint64_t)iters / (uint64_t)c->world;
        st->nccl_bytes = nccl_bytes;
        st->launches = launches;
        st->main_kernel_launches = main_launches;
        st->levels_or_iters = iters;
    } else if (timing) {
        c->t_main.sum_s();
        c->t_merge.sum_s();
        c->t_finish.sum_s();
        c->t_h2d.sum_s();
    }
    return GTS_OK;
}
