// BFS-like algorithms over slotted pages: BFS and SSSP (SURVEY 8(a) a2, a4-a6,
// a10, a12, a13).
//
// Paper: Alg 1 BFS-like path: nextPIDSet holds the pages to visit
// next; per level the kernels run over those pages only, set LV of unvisited
// neighbours to curLevel+1 and mark nextPIDSetGPU; the CPU unions the local
// sets.  Kernels: K_BFS_SP / K_BFS_LP (Alg 2/3).
//
// B200 design: frontier = bitmap (n/8 bytes, L2-resident);
// inside an active page only frontier vertices are expanded (ballot/popc
// compaction, expand.cuh); discovery is exactly-once through atomicOr on the
// visited bitmap (a plain test first, then test-and-set); the level array is
// written once per vertex, coalesced, by the finish kernel from the
// next-frontier bitmap (equivalent to Alg 2 line 18's store of curLevel+1 by
// every discoverer); the next page set is the set of pages whose VID range
// holds a next-frontier bit (segmented OR), computed on the device, so no
// per-edge RVT lookup is needed.  Multi-GPU Strategy-P: next-frontier bitmaps
// are all-gathered over NCCL and OR-ed in the finish kernel (NCCL has no
// bitwise-OR reduction).
#include <cuda_runtime.h>
#include <nccl.h>

#include <algorithm>
#include <array>
#include <cstring>

#include "comm.h"
#include "expand.cuh"
#include "route.cuh"
#include "sweep.cuh"
#include "traverse.h"

namespace gts {

// ------------------------------------------------------------------ ops ---

template <bool W>
struct BfsOp {
    static constexpr bool kReadWeights = false;
    static constexpr bool kWeighted = W;
    static constexpr bool kFastDense = !W;    // plain dense walk (expand.cuh dense_tile_plain)
    static constexpr uint32_t kDense8 = 6;    // dense tiles only at >= 3/4 selected (expand.cuh)
    const uint32_t* cur;
    uint32_t* visited;
    uint32_t* next;
    unsigned long long nedges;
    uint32_t vprefix;          // every vertex below this ID is already visited (no test needed)
    // visited at the start of this level (levels <= the frontier's), nullptr = none: every
    // out-neighbour of such a vertex is already visited (BFS levels differ by at most one
    // along an edge), so expanding its edges discovers nothing -- a dense tile of such
    // vertices can be streamed without selecting the frontier's records
    const uint32_t* vstart;
    uint32_t plain8;           // plain walk when the tile's selected edges are >= plain8/8 of its words
    uint32_t plan_floor;       // whole-page plain plans from this probe floor up (per-tile tests below it)
    __device__ uint32_t fast_floor() const { return vstart ? vprefix : 0u; }
    __device__ bool done(uint32_t v) const { return test_bit(vstart, v); }
    __device__ uint32_t plain_src() const { return 0u; }
    __device__ void plain_edges(uint32_t e) { nedges += e; }   // the frontier's edges in a plain run
    __device__ const uint32_t* frontier() const { return cur; }
    __device__ bool select(uint32_t v) { return test_bit(cur, v); }
    __device__ uint32_t payload(uint32_t, uint32_t deg) {
        nedges += deg;
        return 0u;
    }
    __device__ bool select_lp(uint32_t vid, uint32_t, uint32_t len, uint32_t&) {
        if (!test_bit(cur, vid)) return false;
        if (threadIdx.x == 0) nedges += len;
        return true;
    }
    // (Dropping a frontier vertex whose largest neighbour -- rows are sorted -- lies below
    // the all-visited prefix after one load was measured on RMAT-27: 7.39 vs 7.36 ms; the
    // dependent load per tile costs what the skipped records save.)
    // Alg 2 lines 17-20: if LV[ADJ_VID] = NULL then discover it.  Exactly one
    // thread wins the visited bit and records the vertex in the next frontier.
    // The visited words of the whole edge group are loaded first (independent
    // loads in flight), then tested; the atomic is issued only for clear bits.
    __device__ __forceinline__ void edges(const uint32_t* dst, const uint32_t*, const uint32_t*, const uint32_t*,
                                          const bool* valid) {
        uint32_t vis[kEdgesPerThread];
#pragma unroll
        for (int q = 0; q < kEdgesPerThread; ++q)
            vis[q] = (valid[q] && dst[q] >= vprefix) ? __ldca(visited + (dst[q] >> 5)) : ~0u;
#pragma unroll
        for (int q = 0; q < kEdgesPerThread; ++q) {
            const uint32_t wi = dst[q] >> 5, b = 1u << (dst[q] & 31);
            if (!(vis[q] & b)) {
                if (!(atomicOr(visited + wi, b) & b)) atomicOr(next + wi, b);
            }
        }
    }
    __device__ void end_page() {}
};

template <bool W>
struct SsspOp {
    static constexpr bool kReadWeights = true;
    static constexpr bool kWeighted = W;
    static constexpr bool kSparseSelect = true;   // sparse pages also call select() (expand.cuh)
    const uint32_t* cur;
    uint32_t* dist;
    uint32_t* next;
    unsigned long long nedges;
    bool ovf;
    uint32_t T;                // near-far threshold: only pending vertices with dist <= T are expanded
    // dexp[v] = the distance v's out-edges were last relaxed with (UNREACHED = never).  A
    // pending vertex whose distance has not dropped below it was improved earlier in the
    // round it was expanded in, after which its expansion already used the improved value:
    // expanding it again relaxes nothing.  nullptr = off.  SP vertices only: the slices of
    // an LP vertex run in several CTAs and each must see the same selection.
    uint32_t* dexp;
    __device__ const uint32_t* frontier() const { return cur; }
    __device__ bool select(uint32_t v) {
        if (!test_bit(cur, v)) return false;
        const uint32_t d = __ldcg(dist + v);
        return d <= T && (!dexp || d < __ldcg(dexp + v));
    }
    __device__ uint32_t payload(uint32_t v, uint32_t deg) {
        nedges += deg;
        const uint32_t d = *((volatile uint32_t*)dist + v);
        if (dexp) __stcg(dexp + v, d);
        return d;
    }
    __device__ bool select_lp(uint32_t vid, uint32_t, uint32_t len, uint32_t& pl) {
        if (!test_bit(cur, vid)) return false;
        pl = *((volatile uint32_t*)dist + vid);
        if (pl > T) return false;
        if (threadIdx.x == 0) nedges += len;
        return true;
    }
    // relax (u,v,w): candidates >= 2^32-1 are dropped and flagged (checked
    // exactly after convergence, see sssp_check_kernel)
    __device__ __forceinline__ void edges(const uint32_t* dst, const uint32_t* w, const uint32_t* du,
                                          const uint32_t*, const bool* valid) {
        uint32_t cd[kEdgesPerThread];
#pragma unroll
        for (int q = 0; q < kEdgesPerThread; ++q) cd[q] = valid[q] ? __ldcg(dist + dst[q]) : 0u;
#pragma unroll
        for (int q = 0; q < kEdgesPerThread; ++q) {
            if (!valid[q]) continue;
            const uint64_t nd = (uint64_t)du[q] + w[q];
            if (nd >= (uint64_t)GTS_UNREACHED) {
                ovf = true;
                continue;
            }
            const uint32_t nd32 = (uint32_t)nd;
            if (nd32 < cd[q] && nd32 < atomicMin(dist + dst[q], nd32))
                atomicOr(next + (dst[q] >> 5), 1u << (dst[q] & 31));
        }
    }
    __device__ void end_page() {}
};

// exact overflow test: an edge from a finite vertex into an unreached one (weighted pages)
struct SsspCheckOp {
    static constexpr bool kReadWeights = false;
    static constexpr bool kWeighted = true;
    const uint32_t* dist;
    bool bad;
    __device__ const uint32_t* frontier() const { return nullptr; }
    __device__ bool select(uint32_t v) { return __ldg(dist + v) != GTS_UNREACHED; }
    __device__ uint32_t payload(uint32_t, uint32_t) { return 0u; }
    __device__ bool select_lp(uint32_t vid, uint32_t, uint32_t, uint32_t&) { return __ldg(dist + vid) != GTS_UNREACHED; }
    __device__ __forceinline__ void edges(const uint32_t* dst, const uint32_t*, const uint32_t*, const uint32_t*,
                                          const bool* valid) {
#pragma unroll
        for (int q = 0; q < kEdgesPerThread; ++q)
            if (valid[q] && __ldg(dist + dst[q]) == GTS_UNREACHED) bad = true;
    }
    __device__ void end_page() {}
};

__device__ __forceinline__ void block_add_u64(unsigned long long v, unsigned long long* out) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_down_sync(0xFFFFFFFFu, v, o);
    if ((threadIdx.x & 31) == 0 && v) atomicAdd(out, v);
}

// -------------------------------------------------------------- kernels ---

template <bool W, int M = kMicroTile, int MB = 2>
__global__ void __launch_bounds__(kThreads, MB)
bfs_expand_kernel(PageSet ps, const uint32_t* __restrict__ cur, uint32_t* visited, uint32_t* next,
                  uint32_t* work_ctr, unsigned long long* edges_out, const unsigned int* vprefix_words,
                  uint64_t n, const uint32_t* vstart, uint32_t plain8, uint32_t plan_floor) {
    __shared__ TileSmem sm;
    // all-visited prefix from the previous level's visited_prefix_kernel (device-side,
    // so levels can be enqueued without a host round trip)
    const uint64_t vw = min((uint64_t)*vprefix_words, (n + 31) / 32);
    BfsOp<W> op{cur, visited, next, 0ull, (uint32_t)min(vw * 32, n), vstart, plain8, plan_floor};
    expand_pages<BfsOp<W>, M>(ps, op, sm, work_ctr);
    block_add_u64(op.nedges, edges_out);
}

template <int MB = 2>
__global__ void __launch_bounds__(kThreads, MB)
sssp_expand_kernel(PageSet ps, const uint32_t* __restrict__ cur, uint32_t* dist, uint32_t* next,
                   uint32_t* work_ctr, unsigned long long* edges_out, uint32_t* ovf_flag, uint32_t T, uint32_t* dexp) {
    __shared__ TileSmem sm;
    SsspOp<true> op{cur, dist, next, 0ull, false, T, dexp};
    expand_pages(ps, op, sm, work_ctr);
    block_add_u64(op.nedges, edges_out);
    if (__syncthreads_or(op.ovf) && threadIdx.x == 0) *ovf_flag = 1u;
}

__global__ void __launch_bounds__(kThreads, 2)
sssp_check_kernel(PageSet ps, const uint32_t* __restrict__ dist, uint32_t* work_ctr, uint32_t* bad_flag) {
    __shared__ TileSmem sm;
    SsspCheckOp op{dist, false};
    expand_pages(ps, op, sm, work_ctr);
    if (__syncthreads_or(op.bad) && threadIdx.x == 0) *bad_flag = 1u;
}

// Merge the per-rank next frontiers and count them, over bitmap words [w0, w1)
// (bitmap pointers are biased: word w of the rank's range is ptr[w]).
// gathered != nullptr (Strategy-P / S_BCAST): the world ranks' next bitmaps
// all-gathered [world][gwords]; their OR becomes next and is added to visited.
// gathered == nullptr: next already holds the merged frontier (one rank, or
// Strategy-S after the routed apply).  LV = new_level is written once per newly
// reached vertex when level != nullptr.
__global__ void frontier_finish_kernel(const uint32_t* __restrict__ gathered, int world, uint64_t gwords, uint64_t w0,
                                       uint64_t w1, uint32_t* next, uint32_t* visited, uint32_t* level,
                                       uint32_t new_level, unsigned long long* count, uint32_t* vstart = nullptr) {
    unsigned long long c = 0;
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t w = w0 + (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; w < w1; w += stride) {
        uint32_t bits;
        if (gathered) {
            bits = gathered[w];
            for (int r = 1; r < world; ++r) bits |= gathered[(uint64_t)r * gwords + w];
            next[w] = bits;
            if (visited) visited[w] |= bits;
        } else {
            bits = next[w];
        }
        c += __popc(bits);
        if (vstart && bits) vstart[w] |= bits;    // visited as of the next level's start
        if (level) {
            while (bits) {
                const int b = __ffs(bits) - 1;
                level[w * 32 + b] = new_level;
                bits &= bits - 1;
            }
        }
    }
    block_add_u64(c, count);
}

// SSSP near-far pending set over words [w0, w1) (biased pointers): new pending =
// improved this round (next, or the OR of the all-gathered per-rank bitmaps) +
// pending vertices that were not expanded (dist > T).  Counts the pending
// vertices, those already within T, and the minimum pending distance.
__global__ void sssp_finish_kernel(const uint32_t* __restrict__ gathered, int world, uint64_t gwords, uint64_t w0,
                                   uint64_t w1, const uint32_t* __restrict__ cur, uint32_t* next,
                                   const uint32_t* __restrict__ dist, uint32_t T, unsigned long long* count,
                                   unsigned long long* near, unsigned int* minpend) {
    unsigned long long c = 0, nr = 0;
    uint32_t mn = 0xFFFFFFFFu;
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t w = w0 + (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; w < w1; w += stride) {
        uint32_t bits;
        if (gathered) {
            bits = gathered[w];
            for (int r = 1; r < world; ++r) bits |= gathered[(uint64_t)r * gwords + w];
        } else {
            bits = next[w];
        }
        if (T == 0xFFFFFFFEu) {          // unbounded bucket: every pending distance is within T
            if (gathered) next[w] = bits;
            c += __popc(bits);
            nr += __popc(bits);
            continue;
        }
        uint32_t keep = cur[w] & ~bits;
        while (keep) {
            const int b = __ffs(keep) - 1;
            if (dist[w * 32 + b] > T) bits |= 1u << b;
            keep &= keep - 1;
        }
        next[w] = bits;
        c += __popc(bits);
        uint32_t t = bits;
        while (t) {
            const int b = __ffs(t) - 1;
            const uint32_t dv = dist[w * 32 + b];
            mn = min(mn, dv);
            nr += dv <= T;
            t &= t - 1;
        }
    }
    block_add_u64(c, count);
    block_add_u64(nr, near);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) mn = min(mn, __shfl_down_sync(0xFFFFFFFFu, mn, o));
    if ((threadIdx.x & 31) == 0 && mn != 0xFFFFFFFFu) atomicMin(minpend, mn);
}

// BFS level array from the per-level frontier bitmaps (slot L = the vertices
// first reached at level L; slots are disjoint): LV[v] = the L whose slot holds
// v, UNREACHED if none.  One coalesced pass writes every entry, replacing the
// per-level scattered LV stores and the initial memset (Alg 2 l.18 writes
// curLevel+1 once per discovered vertex; the result is the same array).
// A thread takes one bitmap word (32 vertices): it loads the word of every
// slot (independent loads), folds them into 8 bit planes of the level number,
// and writes its 32 entries as 16-byte stores.  nlev <= 255.
struct LevelPlanes {
    uint32_t reached, p[8];
};

__device__ __forceinline__ LevelPlanes level_planes(const uint32_t* __restrict__ slots, uint32_t nlev, uint64_t words,
                                                    uint64_t w) {
    LevelPlanes lp{0u, {0u, 0u, 0u, 0u, 0u, 0u, 0u, 0u}};
#pragma unroll 8
    for (uint32_t L = 0; L < nlev; ++L) {
        const uint32_t x = __ldg(slots + (uint64_t)L * words + w);
        lp.reached |= x;
#pragma unroll
        for (int k = 0; k < 8; ++k)
            if ((L >> k) & 1u) lp.p[k] |= x;
    }
    return lp;
}

__device__ __forceinline__ uint32_t level_of_bit(const LevelPlanes& lp, int b) {
    uint32_t l = 0;
#pragma unroll
    for (int k = 0; k < 8; ++k) l |= ((lp.p[k] >> b) & 1u) << k;
    return l;
}

__global__ void level_fill_kernel(uint32_t* level, const uint32_t* __restrict__ slots, uint32_t nlev, uint64_t words,
                                  uint64_t n) {
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t w = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; w < words; w += stride) {
        const LevelPlanes lp = level_planes(slots, nlev, words, w);
        const uint64_t v0 = w * 32;
        if (v0 + 32 <= n) {
            uint4* o = reinterpret_cast<uint4*>(level + v0);
#pragma unroll
            for (int q = 0; q < 8; ++q) {
                uint32_t e[4];
#pragma unroll
                for (int k = 0; k < 4; ++k) {
                    const int b = 4 * q + k;
                    e[k] = ((lp.reached >> b) & 1u) ? level_of_bit(lp, b) : GTS_UNREACHED;
                }
                o[q] = make_uint4(e[0], e[1], e[2], e[3]);
            }
        } else {
            for (int b = 0; v0 + b < n; ++b) level[v0 + b] = ((lp.reached >> b) & 1u) ? level_of_bit(lp, b) : GTS_UNREACHED;
        }
    }
}

// Degree-ordered graphs: the same levels as bytes (0xFF = unreached; fewer than
// 255 levels; the byte array holds words * 32 entries), then the caller-order
// output gathered from that n-byte array (mostly L2-resident) instead of from
// the 4n-byte LV.
__global__ void level_fill8_kernel(uint8_t* lv8, const uint32_t* __restrict__ slots, uint32_t nlev, uint64_t words) {
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t w = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; w < words; w += stride) {
        const LevelPlanes lp = level_planes(slots, nlev, words, w);
        uint32_t e[8];
#pragma unroll
        for (int q = 0; q < 8; ++q) {
            uint32_t x = 0;
#pragma unroll
            for (int k = 0; k < 4; ++k) {
                const int b = 4 * q + k;
                const uint32_t l = ((lp.reached >> b) & 1u) ? level_of_bit(lp, b) : 0xFFu;
                x |= l << (8 * k);
            }
            e[q] = x;
        }
        uint4* o = reinterpret_cast<uint4*>(lv8 + w * 32);
        o[0] = make_uint4(e[0], e[1], e[2], e[3]);
        o[1] = make_uint4(e[4], e[5], e[6], e[7]);
    }
}

// Fewer than 15 levels (every RMAT / power-law traversal): 4-bit levels, 0xF =
// unreached.  The n/2-byte array (67 MB at RMAT-27) stays in L2 for the gather.
__global__ void level_fill4_kernel(uint8_t* lv4, const uint32_t* __restrict__ slots, uint32_t nlev, uint64_t words) {
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t w = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; w < words; w += stride) {
        const LevelPlanes lp = level_planes(slots, nlev, words, w);
        // bit b of plane k becomes bit k of nibble b: spread each byte of a plane to every
        // fourth bit (bit i -> bit 4i) and shift it into place; unreached nibbles are 0xF
        auto spread = [](uint32_t x) {         // 8 bits -> bits 0, 4, ..., 28
            x = (x | (x << 12)) & 0x000F000Fu;
            x = (x | (x << 6)) & 0x03030303u;
            return (x | (x << 3)) & 0x11111111u;
        };
        uint32_t e[4];
#pragma unroll
        for (int q = 0; q < 4; ++q) {
            const int sh = 8 * q;
            e[q] = spread((lp.p[0] >> sh) & 0xFFu) | spread((lp.p[1] >> sh) & 0xFFu) << 1 |
                   spread((lp.p[2] >> sh) & 0xFFu) << 2 | spread((lp.p[3] >> sh) & 0xFFu) << 3 |
                   spread(~(lp.reached >> sh) & 0xFFu) * 0xFu;
        }
        reinterpret_cast<uint4*>(lv4)[w] = make_uint4(e[0], e[1], e[2], e[3]);
    }
}

__global__ void gather4_kernel(uint32_t* out, const uint8_t* __restrict__ lv4, const uint32_t* __restrict__ idx,
                               uint64_t n) {
    gather_x4(out, idx, n, [&](uint32_t i) {
        const uint32_t l = (__ldg(lv4 + (i >> 1)) >> (4 * (i & 1))) & 0xFu;
        return l == 0xFu ? GTS_UNREACHED : l;
    });
}

__global__ void gather8_kernel(uint32_t* out, const uint8_t* __restrict__ lv8, const uint32_t* __restrict__ idx,
                               uint64_t n) {
    gather_x4(out, idx, n, [&](uint32_t i) {
        const uint32_t l = __ldg(lv8 + i);
        return l == 0xFFu ? GTS_UNREACHED : l;
    });
}

// Length of the all-visited prefix of the bitmap, in words: the first word that
// is not all ones.  On a degree-ordered graph the low IDs are the hubs and are
// reached in the first levels, so later levels skip the visited test of every
// edge into that prefix.
__global__ void visited_prefix_kernel(const uint32_t* __restrict__ visited, uint64_t words, unsigned int* first) {
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t w = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; w < words; w += stride) {
        const bool hole = visited[w] != 0xFFFFFFFFu;
        const uint32_t m = __ballot_sync(__activemask(), hole);
        if (m && (threadIdx.x & 31) == __ffs(m) - 1) atomicMin(first, (unsigned int)w);
        if (__any_sync(__activemask(), hole)) break;   // later words of this thread cannot be smaller
    }
}

// Next page set (nextPIDSet, Alg 1 lines 29-30): the pages among
// `pages` (this rank's) whose VID range [START_VID, START_VID + nslots) has a
// bit set in `bits`.  One warp per page.
__global__ void frontier_pages_kernel(const uint32_t* __restrict__ bits, const uint32_t* __restrict__ rvt_start,
                                      const uint32_t* __restrict__ nslots, const uint32_t* __restrict__ pages,
                                      uint32_t npages, uint32_t* out_list, uint32_t* out_count) {
    const int lane = threadIdx.x & 31;
    const uint32_t warps = (gridDim.x * blockDim.x) >> 5;
    for (uint32_t i = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; i < npages; i += warps) {
        const uint32_t p = pages ? pages[i] : i;
        const uint64_t lo = rvt_start[p], hi = lo + nslots[p];   // [lo, hi)
        const uint64_t w0 = lo >> 5, w1 = (hi - 1) >> 5;
        bool any = false;
        for (uint64_t w = w0 + lane; w <= w1; w += 32) {
            uint32_t m = bits[w];
            if (w == w0) m &= 0xFFFFFFFFu << (lo & 31);
            if (w == w1 && ((hi & 31) != 0)) m &= 0xFFFFFFFFu >> (32 - (hi & 31));
            any |= m != 0;
        }
        if (__any_sync(0xFFFFFFFFu, any) && lane == 0) out_list[atomicAdd(out_count, 1u)] = p;
    }
}

__global__ void set_source_kernel(uint32_t* value, uint32_t* visited, uint32_t* cur, uint64_t src) {
    value[src] = 0;
    if (visited) visited[src >> 5] |= 1u << (src & 31);
    cur[src >> 5] |= 1u << (src & 31);
}

// ---------------------------------------------------------------- driver ---

struct Counters {               // device scratch, slot kCtr
    uint32_t work;
    uint32_t list_count;
    unsigned long long count;
    unsigned long long edges;
    uint32_t flag;
    uint32_t flag2;
    unsigned long long near;       // SSSP: pending vertices within the threshold
    unsigned int minpend;          // SSSP: minimum pending distance
    unsigned int vprefix_words;    // BFS: all-visited prefix of the bitmap (words)
};

enum { kBufValue = 0, kBufVisited, kBufCur, kBufNext, kBufList, kBufCtr, kBufGather, kBufLvSlots, kBufLv8, kBufLvCnt,
       kBufDexp, kBufVstart };

// deliver() for byte levels of a degree-ordered graph: out[v] = lv8[new_of_old[v]]
static int deliver_levels8(Context* c, const Graph* g, const uint8_t* lv8, bool nibbles, void* out,
                           uint32_t out_location) {
    const uint64_t n = g->n;
    uint32_t* dst;
    if (out_location == GTS_OUT_DEVICE) dst = static_cast<uint32_t*>(out);
    else GTS_TRY(c->buf(72, n * 4, (void**)&dst));     // deliver()'s staging slot
    if (nibbles) gather4_kernel<<<c->num_sms * 8, 256, 0, c->stream>>>(dst, lv8, c->dg.new_of_old, n);
    else gather8_kernel<<<c->num_sms * 8, 256, 0, c->stream>>>(dst, lv8, c->dg.new_of_old, n);
    GTS_CUDA(cudaGetLastError());
    if (out_location == GTS_OUT_DEVICE) {
        GTS_CUDA(cudaStreamSynchronize(c->stream));
        return GTS_OK;
    }
    return copy_out(c, dst, out, n * 4, out_location);
}

// pages holding vertex v among this rank's pages (Alg 1 line 5: "page ID containing start vertex")
static std::vector<uint32_t> pages_of_vertex(const Graph* g, const DevGraph& d, int rank, uint64_t v) {
    std::vector<uint32_t> out;
    auto it = std::upper_bound(g->start_vid.begin(), g->start_vid.end(), (uint32_t)v);
    int64_t p = (int64_t)(it - g->start_vid.begin()) - 1;
    if (p < 0) return out;
    int64_t a = p, b = p;
    if (g->kind[p] == GTS_PAGE_LP) {
        a = g->lp_first[p];
        b = g->lp_last[p];
    }
    for (int64_t q = a; q <= b; ++q)
        if (d.h_owner[q] == rank) out.push_back((uint32_t)q);
    return out;
}

static PageSet resident_set(Context* c, const Graph* g, const uint32_t* list, const uint32_t* d_count) {
    PageSet ps;
    ps.base = c->dg.pages;
    ps.list = list;
    ps.loc = c->dg.loc;
    ps.d_count = d_count;
    ps.count = 0;
    ps.page_bytes = g->page_bytes;
    ps.mode = c->dg.all_local ? kAddrByPid : kAddrByLoc;
    ps.entry_encoding = g->entry_encoding;
    ps.rvt_start = c->dg.rvt_start;
    return ps;
}

// One rank (world 1, no virtual ranks): the tuned single-GPU path (level
// slots, batched levels, degree-ordered byte levels, LP slicing, page cache).
static int traverse_single(gts_context* c, const gts_graph* g, uint64_t src, const gts_run_config& rc, uint32_t* out,
                           gts_run_stats* st, int algo, double t_start, bool streamed, double upload_s) {
    const uint64_t n = g->n, words = (n + 31) / 32;
    const bool timing = rc.flags & GTS_RUN_TIMING;
    uint32_t *value, *visited = nullptr, *cur, *next, *list;
    Counters* ctr;
    GTS_TRY(c->buf(kBufValue, n * 4, (void**)&value));
    if (algo == kBFS) GTS_TRY(c->buf(kBufVisited, words * 4, (void**)&visited));
    GTS_TRY(c->buf(kBufCur, words * 4, (void**)&cur));
    GTS_TRY(c->buf(kBufNext, words * 4, (void**)&next));
    GTS_TRY(c->buf(kBufList, std::max<uint64_t>(g->num_pages, 1) * 4, (void**)&list));
    GTS_TRY(c->buf(kBufCtr, sizeof(Counters), (void**)&ctr));
    cudaStream_t s = c->stream;
    // micro-level technique inside each page (GTS_MICRO_*, App E): BFS only
    uint32_t micro = (rc.flags & GTS_MICRO_MASK) >> 8;
    if (micro == (GTS_MICRO_TILE >> 8)) micro = kMicroTile;
    if (micro > kMicroHybrid) return fail(GTS_EINVAL, "unknown GTS_MICRO value");
    if (algo == kSSSP && micro) return fail(GTS_EUNSUPPORTED, "GTS_MICRO_* techniques apply to gts_bfs and gts_pagerank");
    // BFS, unweighted degree-ordered pages: visited as of the start of each level, for the
    // plain dense walk (BfsOp::vstart): a copy of visited after the source is set, then OR-ed
    // with each level's new frontier by frontier_finish_kernel
    uint32_t* vstart = nullptr;
    if (algo == kBFS && g->ordered && !g->weighted && micro == kMicroTile)
        GTS_TRY(c->buf(kBufVstart, words * 4, (void**)&vstart));
    // tiles whose selected edges are >= 3/8 of their words take the plain walk (RMAT-27 BFS
    // kernels 6.57 ms against 6.65 at 6/8, 6.60 at 4/8, 6.58 at 2/8, 6.65 at 1/8)
    constexpr uint32_t plain8 = 3;
    // BFS decides per tile, after the tile's own setup: whole-page plans (expand.cuh
    // plan_plain_tiles) measured slower at every floor (RMAT-27 BFS kernels 6.53 ms per tile,
    // 6.73-6.92 ms with plans from floors of 8 M down to 0)
    constexpr uint32_t plan_floor = 0xFFFFFFFFu;
    uint32_t* dexp = nullptr;            // SSSP: distance of each vertex's last expansion (SsspOp)
    if (algo == kSSSP) {     // RMAT-27: 4.51 G -> 3.12 G relaxed edges, kernels 33.1 -> 26.1 ms
        GTS_TRY(c->buf(kBufDexp, n * 4, (void**)&dexp));
        GTS_CUDA(cudaMemsetAsync(dexp, 0xFF, n * 4, s));
    }
    // BFS level slots: the frontier of level L lives in slot L of a K-slot bitmap
    // store, and LV is written once at the end by level_fill_kernel.  A traversal
    // deeper than K levels fills LV from the slots and continues with the
    // ping-pong frontiers, writing LV per level in frontier_finish_kernel.
    // gts_run_config.bfs_level_slots = K (GTS_OFF: per-level LV writes throughout); default 32,
    // capped at 1 GiB.
    uint32_t K = 0;
    uint32_t* lvb = nullptr;
    if (algo == kBFS) {
        K = rc.bfs_level_slots == GTS_OFF ? 0u : rc.bfs_level_slots ? rc.bfs_level_slots : 32u;
        K = (uint32_t)std::min<uint64_t>(std::min<uint64_t>(K, 255), (1ull << 30) / (words * 4));
        if (K < 3) K = 0;
        if (K) {
            GTS_TRY(c->buf(kBufLvSlots, (size_t)K * words * 4, (void**)&lvb));
            cur = lvb;
            next = lvb + words;
        }
    }
    bool slots = K > 0;
    if (!slots) GTS_CUDA(cudaMemsetAsync(value, 0xFF, n * 4, s));
    if (visited) GTS_CUDA(cudaMemsetAsync(visited, 0, words * 4, s));
    GTS_CUDA(cudaMemsetAsync(cur, 0, words * 4, s));
    GTS_CUDA(cudaMemsetAsync(next, 0, words * 4, s));
    GTS_CUDA(cudaMemsetAsync(ctr, 0, sizeof(Counters), s));
    src = map_src(g, src);
    set_source_kernel<<<1, 1, 0, s>>>(value, visited, cur, src);
    if (vstart) GTS_CUDA(cudaMemcpyAsync(vstart, visited, words * 4, cudaMemcpyDeviceToDevice, s));
    uint64_t launches = 1, main_launches = 0;
    std::vector<uint32_t> l0 = pages_of_vertex(g, c->dg, c->rank, src);
    uint32_t* hs = (uint32_t*)c->h_small;
    hs[0] = (uint32_t)l0.size();
    if (!l0.empty()) GTS_CUDA(cudaMemcpyAsync(list, l0.data(), l0.size() * 4, cudaMemcpyHostToDevice, s));
    GTS_CUDA(cudaMemcpyAsync(&ctr->list_count, hs, 4, cudaMemcpyHostToDevice, s));

    using BfsKern = decltype(&bfs_expand_kernel<false, kMicroTile>);
    static const BfsKern bfs_k[2][4] = {
        {bfs_expand_kernel<false, kMicroTile>, bfs_expand_kernel<false, kMicroEdge>,
         bfs_expand_kernel<false, kMicroVertex>, bfs_expand_kernel<false, kMicroHybrid>},
        {bfs_expand_kernel<true, kMicroTile>, bfs_expand_kernel<true, kMicroEdge>,
         bfs_expand_kernel<true, kMicroVertex>, bfs_expand_kernel<true, kMicroHybrid>}};
    BfsKern bfs_kern = bfs_k[g->weighted ? 1 : 0][micro];
    // three 512-thread CTAs per SM (40 registers): the per-tile barriers of one CTA are
    // covered by the other two (RMAT-27 BFS kernels 10.25 -> 9.26 ms against two)
    if (micro == kMicroTile)
        bfs_kern = g->weighted ? bfs_expand_kernel<true, kMicroTile, 3> : bfs_expand_kernel<false, kMicroTile, 3>;
    const uint32_t hybrid_deg = rc.hybrid_deg ? rc.hybrid_deg : 8u;
    // three 512-thread CTAs per SM for the SSSP expansion: with the interleaved (adj, w)
    // records it fits 40 registers (20 bytes spilled) -- RMAT-27 33.6 vs 34.2 ms for two
    auto sssp_kern = sssp_expand_kernel<3>;
    const void* kexp = algo == kBFS ? (const void*)bfs_kern : (const void*)sssp_kern;
    int grid = 0;
    GTS_TRY(sms_grid(c, kexp, kThreads, 0, &grid));
    const int fin_grid = c->num_sms * 4;
    uint64_t pages_processed = l0.size();
    uint32_t levels = 0;
    Counters h;
    SweepStats ss;
    std::vector<uint32_t> h_list = l0;             // streamed mode: this level's pages on the host (ascending)
    const bool cached = streamed && rc.cache_mib > 0;
    // SSSP near-far bucketing: expand only pending vertices with dist <= T; T
    // advances by delta past the nearest pending distance when no pending vertex
    // is within it.  Label-correcting, so any delta gives the exact distances.
    // Default unbounded (plain frontier Bellman-Ford): on RMAT-27 delta 16 / 64 /
    // 256 / unbounded measured 71 / 49 / 38 / 36 ms -- low-diameter power-law
    // graphs waste few relaxations.  gts_run_config.sssp_delta selects a bucket width.
    const uint64_t delta = rc.sssp_delta ? rc.sssp_delta : 0xFFFFFFFEull;
    uint32_t T = algo == kSSSP ? (uint32_t)std::min<uint64_t>(delta, 0xFFFFFFFEull) : 0xFFFFFFFEu;
    // Persisting-L2 window on the structure every edge probes: SSSP on degree-ordered
    // pages the dense head [0, W) of dist (the most relaxed entries), BFS the visited
    // bitmap.  It also replaces lines an earlier PageRank call left persisting.
    // gts_run_config.l2_persist_mib (0 = 96 MiB, GTS_OFF = none).
    bool persist = false;
    if (!streamed && (algo == kBFS || g->ordered)) {
        const size_t want = std::min<size_t>((size_t)l2_persist_mib(rc) << 20, algo == kBFS ? words * 4 : n * 4);
        if (want > 0) {
            GTS_TRY(persist_window(c, s, algo == kBFS ? (void*)visited : (void*)value, want));
            persist = true;
        }
    }
    // BFS on resident pages, one rank: levels are enqueued levels_per_sync (default 8) at
    // a time without a host round trip (per-level new-vertex counts and page-list counts go
    // to device arrays; the levels after the last non-empty one run on an empty frontier)
    // SSSP with an unbounded bucket (the default: T never moves) batches its rounds the same way,
    // each round's pending count and page-list count going to a 64-entry ring
    const bool sssp_batch = algo == kSSSP && !streamed && !cached && rc.sssp_delta == 0;
    const uint32_t B = ((algo == kBFS && K > 0) || sssp_batch) && !streamed
                           ? std::min<uint32_t>(rc.levels_per_sync ? rc.levels_per_sync : 8u, 32u) : 1u;
    constexpr uint32_t kRing = 64;
    unsigned long long* ring_cnt = nullptr;          // SSSP batched rounds: [kRing] pending counts
    uint32_t* ring_pages = nullptr;                  // [kRing] pages in the next round's list
    if (sssp_batch) {
        GTS_TRY(c->buf(kBufLvCnt, (size_t)kRing * 12, (void**)&ring_cnt));
        ring_pages = reinterpret_cast<uint32_t*>(ring_cnt + kRing);
    }
    unsigned long long* lvl_cnt = nullptr;           // [K] new vertices per level (BFS)
    uint32_t* lvl_pages = nullptr;                   // [K] pages in the list of level L
    if (algo == kBFS) {
        const uint32_t nl = std::max<uint32_t>(K, 1) + 1;
        GTS_TRY(c->buf(kBufLvCnt, (size_t)nl * 12, (void**)&lvl_cnt));
        lvl_pages = reinterpret_cast<uint32_t*>(lvl_cnt + nl);
        GTS_CUDA(cudaMemsetAsync(lvl_cnt, 0, (size_t)nl * 12, s));
    }
    std::vector<unsigned long long> h_cnt;
    std::vector<uint32_t> h_pages;
    uint32_t synced = 0;                             // levels whose counts the host has read
    for (uint32_t L = 0;; ++L) {
        auto launch = [&](const PageSet& ps, int cap) -> int {
                                GTS_CUDA(cudaMemsetAsync(&ctr->work, 0, 4, s));
                                std::pair<cudaEvent_t, cudaEvent_t> ev;
                                if (timing) { ev = c->t_main.next(); cudaEventRecord(ev.first, s); }
                                PageSet p2 = ps;
                                p2.hybrid_deg = hybrid_deg;
                                // few pages in this level (e.g. the source hub's LPs): slice LPs so
                                // every CTA gets work, decided on the device
                                p2.split = 0u;
                                const int gl = std::min(grid, cap);
                                if (algo == kBFS) {
                                    bfs_kern<<<gl, kThreads, 0, s>>>(
                                        p2, cur, visited, next, &ctr->work, &ctr->edges, &ctr->vprefix_words, n,
                                        vstart, plain8, plan_floor);
                                } else
                                    sssp_kern<<<gl, kThreads, 0, s>>>(
                                        p2, cur, value, next, &ctr->work, &ctr->edges, &ctr->flag, T, dexp);
                                if (timing) cudaEventRecord(ev.second, s);
                                GTS_CUDA(cudaGetLastError());
                                ++main_launches;
                                return GTS_OK;
                            };
        if (cached) GTS_TRY(sweep_pages_cached(c, g, rc, h_list, list, launch, &ss));
        else GTS_TRY(sweep_pages(c, g, rc, streamed, &h_list, list, (uint32_t)h_list.size(), &ctr->list_count,
                                 launch, &ss));
        std::pair<cudaEvent_t, cudaEvent_t> ev;
        if (timing) { ev = c->t_finish.next(); cudaEventRecord(ev.first, s); }
        GTS_CUDA(cudaMemsetAsync(&ctr->count, 0, 8, s));
        GTS_CUDA(cudaMemsetAsync(&ctr->list_count, 0, 4, s));
        if (algo == kBFS) {
            frontier_finish_kernel<<<fin_grid, 256, 0, s>>>(nullptr, 1, words, 0, words, next, visited,
                                                            slots ? nullptr : value, L + 1,
                                                            L < K ? lvl_cnt + L : &ctr->count, vstart);
            GTS_CUDA(cudaMemsetAsync(&ctr->vprefix_words, 0xFF, 4, s));
            visited_prefix_kernel<<<fin_grid, 256, 0, s>>>(visited, words, &ctr->vprefix_words);
            ++launches;
        } else {
            GTS_CUDA(cudaMemsetAsync(&ctr->near, 0, 8, s));
            GTS_CUDA(cudaMemsetAsync(&ctr->minpend, 0xFF, 4, s));
            unsigned long long* cnt = &ctr->count;
            if (sssp_batch) {
                cnt = ring_cnt + (L % kRing);
                GTS_CUDA(cudaMemsetAsync(cnt, 0, 8, s));
            }
            sssp_finish_kernel<<<fin_grid, 256, 0, s>>>(nullptr, 1, words, 0, words, cur, next, value, T,
                                                        cnt, &ctr->near, &ctr->minpend);
        }
        frontier_pages_kernel<<<fin_grid, 256, 0, s>>>(next, c->dg.rvt_start, c->dg.nslots,
                                                       c->dg.all_local ? nullptr : c->dg.local_list,
                                                       c->dg.all_local ? (uint32_t)g->num_pages : c->dg.n_local,
                                                       list, &ctr->list_count);
        if (timing) cudaEventRecord(ev.second, s);
        launches += 2;
        GTS_CUDA(cudaGetLastError());
        if (algo == kBFS && L < K)                    // pages of level L+1's list (lvl_pages has K+1 entries)
            GTS_CUDA(cudaMemcpyAsync(lvl_pages + L + 1, &ctr->list_count, 4, cudaMemcpyDeviceToDevice, s));
        if (sssp_batch)
            GTS_CUDA(cudaMemcpyAsync(ring_pages + (L % kRing), &ctr->list_count, 4, cudaMemcpyDeviceToDevice, s));
        ++levels;
        // host round trip: every level (near-far SSSP, streamed), else every B levels and
        // before the level slots run out
        // the batches after the first are half as long: a traversal that outlives its first
        // batch is usually in its tail (RMAT-27 SSSP: 11 rounds ran as 8 + 8, five of them on
        // an empty frontier, ~80 us each; now 8 + 4)
        const uint32_t B2 = std::max(1u, B / 2);
        const bool sync = B == 1 || (L + 1 <= B ? (L + 1) % B == 0 : (L + 1 - B) % B2 == 0) ||
                          (algo == kBFS && !(slots && L + 3 < K));
        if (!sync) {
            if (slots && L + 2 < K) {
                cur = next;
                next = lvb + (uint64_t)(L + 2) * words;
                GTS_CUDA(cudaMemsetAsync(next, 0, words * 4, s));
                continue;
            }
            if (sssp_batch) {
                std::swap(cur, next);
                GTS_CUDA(cudaMemsetAsync(next, 0, words * 4, s));
                continue;
            }
        }
        GTS_CUDA(cudaMemcpyAsync(&h, ctr, sizeof(Counters), cudaMemcpyDeviceToHost, s));
        std::vector<unsigned long long> r_cnt;
        std::vector<uint32_t> r_pages;
        if (sssp_batch) {
            r_cnt.resize(kRing);
            r_pages.resize(kRing);
            GTS_CUDA(cudaMemcpyAsync(r_cnt.data(), ring_cnt, kRing * 8, cudaMemcpyDeviceToHost, s));
            GTS_CUDA(cudaMemcpyAsync(r_pages.data(), ring_pages, kRing * 4, cudaMemcpyDeviceToHost, s));
        }
        if (algo == kBFS && L < K) {
            h_cnt.resize(L + 1);
            h_pages.resize(L + 2);
            GTS_CUDA(cudaMemcpyAsync(h_cnt.data() + synced, lvl_cnt + synced, (size_t)(L + 1 - synced) * 8,
                                     cudaMemcpyDeviceToHost, s));
            GTS_CUDA(cudaMemcpyAsync(h_pages.data() + synced + 1, lvl_pages + synced + 1, (size_t)(L + 1 - synced) * 4,
                                     cudaMemcpyDeviceToHost, s));
        }
        GTS_CUDA(cudaStreamSynchronize(s));
        if (algo == kBFS && L < K) {
            bool done = false;
            for (uint32_t l = synced; l <= L; ++l) {
                if (h_cnt[l] == 0) {                  // level l discovered nothing: BFS ends there
                    levels = l + 1;
                    done = true;
                    break;
                }
                pages_processed += h_pages[l + 1];
            }
            synced = L + 1;
            h.count = done ? 0 : h_cnt[L];
            h.list_count = h_pages[L + 1];
            if (done) break;
        }
        if (sssp_batch) {                         // rounds synced..L of the batch
            bool done = false;
            for (uint32_t l = synced; l <= L; ++l) {
                if (r_cnt[l % kRing] == 0) {         // round l left nothing pending: SSSP ends there
                    levels = l + 1;
                    done = true;
                    break;
                }
                if (l < L) pages_processed += r_pages[l % kRing];
            }
            synced = L + 1;
            h.count = done ? 0 : r_cnt[L % kRing];
            h.list_count = r_pages[L % kRing];
        }
        if (h.count == 0) break;
        if (algo == kSSSP && !sssp_batch && h.near == 0) {   // nothing pending within T: open the next bucket
            const uint64_t nt = (uint64_t)h.minpend + delta;
            T = (uint32_t)std::min<uint64_t>(nt, 0xFFFFFFFEull);
        }
        if (algo != kBFS || L >= K) pages_processed += h.list_count;
        if (streamed) {                          // the host drives the copies: fetch and sort the page set
            h_list.resize(h.list_count);
            if (h.list_count) {
                GTS_CUDA(cudaMemcpyAsync(h_list.data(), list, h.list_count * 4ull, cudaMemcpyDeviceToHost, s));
                GTS_CUDA(cudaStreamSynchronize(s));
                std::sort(h_list.begin(), h_list.end());
                GTS_CUDA(cudaMemcpyAsync(list, h_list.data(), h.list_count * 4ull, cudaMemcpyHostToDevice, s));
                GTS_CUDA(cudaStreamSynchronize(s));
            }
        }
        if (slots && L + 2 < K) {                // next level's frontier in the next slot
            cur = next;
            next = lvb + (uint64_t)(L + 2) * words;
        } else {
            if (slots) {                          // out of slots: LV for levels 0..L+1 now
                level_fill_kernel<<<fin_grid, 256, 0, s>>>(value, lvb, L + 2, words, n);
                GTS_CUDA(cudaGetLastError());
                ++launches;
                slots = false;
                GTS_TRY(c->buf(kBufNext, words * 4, (void**)&next));
                cur = lvb + (uint64_t)(L + 1) * words;
                std::swap(cur, next);             // (swapped back below)
            }
            std::swap(cur, next);
        }
        GTS_CUDA(cudaMemsetAsync(next, 0, words * 4, s));
    }
    uint8_t* lv8 = nullptr;
    const bool nib = levels < 15;
    if (slots && g->ordered && nib) {
        GTS_TRY(c->buf(kBufLv8, words * 32, (void**)&lv8));
        level_fill4_kernel<<<2 * fin_grid, 256, 0, s>>>(lv8, lvb, levels, words);
        GTS_CUDA(cudaGetLastError());
        launches += 2;
    } else if (slots && g->ordered && levels < 255) {
        GTS_TRY(c->buf(kBufLv8, words * 32, (void**)&lv8));
        level_fill8_kernel<<<fin_grid, 256, 0, s>>>(lv8, lvb, levels, words);
        GTS_CUDA(cudaGetLastError());
        launches += 2;
    } else if (slots) {
        level_fill_kernel<<<fin_grid, 256, 0, s>>>(value, lvb, levels, words, n);
        GTS_CUDA(cudaGetLastError());
        ++launches;
    }
    if (persist) GTS_TRY(persist_window(c, s, nullptr, 0));
    if (algo == kSSSP && h.flag) {
        // exact overflow test (see SsspOp::edges): sweep all local pages once
        GTS_CUDA(cudaMemsetAsync(&ctr->flag2, 0, 4, s));
        int g2 = 0;
        GTS_TRY(sms_grid(c, (const void*)sssp_check_kernel, kThreads, 0, &g2));
        GTS_TRY(sweep_pages(c, g, rc, streamed, &c->dg.h_local_list,
                            (c->dg.all_local && !streamed) ? nullptr : c->dg.local_list, c->dg.n_local, nullptr,
                            [&](const PageSet& ps, int cap) -> int {
                                GTS_CUDA(cudaMemsetAsync(&ctr->work, 0, 4, s));
                                sssp_check_kernel<<<std::min(g2, cap), kThreads, 0, s>>>(ps, value, &ctr->work,
                                                                                        &ctr->flag2);
                                GTS_CUDA(cudaGetLastError());
                                ++launches;
                                return GTS_OK;
                            }, &ss));
        uint32_t bad = 0;
        GTS_CUDA(cudaMemcpyAsync(&bad, &ctr->flag2, 4, cudaMemcpyDeviceToHost, s));
        GTS_CUDA(cudaStreamSynchronize(s));
        if (bad) return fail(GTS_EOVERFLOW, "an SSSP distance reaches 2^32-1");
    }
    if (lv8) GTS_TRY(deliver_levels8(c, g, lv8, nib, out, rc.out_location));
    else GTS_TRY(deliver(c, g, value, out, rc.out_location, false));
    if (st) {
        std::memset(st, 0, sizeof(*st));
        st->wall_s = now_s() - t_start;
        st->upload_s = upload_s;
        if (timing) {
            st->main_kernel_s = c->t_main.sum_s();
            st->merge_s = c->t_merge.sum_s();
            st->finish_s = c->t_finish.sum_s();
        }
        st->pages_processed = pages_processed;
        st->h2d_bytes = ss.h2d_bytes;
        st->cache_hits = ss.cache_hits;
        st->cache_misses = ss.cache_misses;
        if (timing) st->h2d_s = c->t_h2d.sum_s();
        st->edges_traversed = h.edges;
        st->wa_bytes = (uint64_t)n * 4 + (uint64_t)(algo == kBFS ? 3 : 2) * words * 4;
        st->launches = launches + main_launches;
        st->main_kernel_launches = main_launches;
        st->levels_or_iters = levels;
    } else if (timing) {
        c->t_main.sum_s();
        c->t_merge.sum_s();
        c->t_finish.sum_s();
        c->t_h2d.sum_s();
    }
    return GTS_OK;
}

// ------------------------------------------------------- multi-rank path ---
// N ranks (real, one per process, or virtual on one GPU; comm.h), Strategy-P,
// Strategy-S with routed updates, or the paper-literal S_BCAST:
//   P       pages h(j) = j mod N, WA replicated; per level every rank expands
//           its frontier pages into its own next bitmap, the bitmaps are
//           all-gathered and OR-ed (NCCL has no bitwise OR);
//           SSSP also all-reduces dist with min.
//   S       rank r owns WA [lo, hi) and the pages whose sources lie in it; a
//           remote destination becomes a message to its owner (BFS: dst,
//           deduplicated per sender by a sent bitmap; SSSP: (dst, dist);
//           WCC: (dst, label)), exchanged with grouped send/recv and applied
//           by the owner; frontier counts are all-reduced.
//   S_BCAST every rank expands every frontier page but applies only updates
//           into its own range; the ranges are merged as under P.
// WCC under S is push-only min-label propagation on GTS_BUILD_SYMMETRIC pages
// (each edge is stored at both endpoints, so the owner of either endpoint
// pushes along it; SURVEY 8(e) WCC caveat): the result, the minimum VID of
// each weakly connected component, is the union-find result.

enum { kDstAll = 0, kDstRoute = 1, kDstDrop = 2 };   // remote destinations: (none under P), route, drop

__device__ __forceinline__ bool in_range(uint32_t v, uint64_t lo, uint64_t hi) { return (uint64_t)v - lo < hi - lo; }

// GTS_ROUTE_PEER: every owner's WA as seen by this rank (biased pointers: absolute
// VIDs / bitmap words), so a remote update is one atomic over peer memory
struct PeerWA {
    uint32_t* val[kMaxRanks];   // LV / dist / label
    uint32_t* vis[kMaxRanks];   // BFS visited bitmap
    uint32_t* nxt[kMaxRanks];   // next-frontier bitmap of this level
};

template <bool W>
struct MBfsOp {
    static constexpr bool kReadWeights = false;
    static constexpr bool kWeighted = W;
    static constexpr uint32_t kDense8 = 6;
    const uint32_t* cur;       // biased bitmaps (word w of the rank's range at ptr[w])
    uint32_t* visited;
    uint32_t* next;
    uint32_t* sent;            // Strategy-S: remote vertices already sent by this rank (full n bits)
    unsigned long long nedges;
    uint64_t lo, hi;
    int mode;
    RouteOut ro;
    int direct;                // GTS_ROUTE_PEER
    PeerWA pw;
    __device__ const uint32_t* frontier() const { return cur; }
    __device__ bool select(uint32_t v) { return test_bit(cur, v); }
    __device__ uint32_t payload(uint32_t, uint32_t deg) {
        nedges += deg;
        return 0u;
    }
    __device__ bool select_lp(uint32_t vid, uint32_t, uint32_t len, uint32_t&) {
        if (!test_bit(cur, vid)) return false;
        if (threadIdx.x == 0) nedges += len;
        return true;
    }
    // Alg 2 lines 17-20 for local destinations (exactly-once discovery through the
    // visited bit); remote ones go to their owner once per traversal (sent bit).
    __device__ __forceinline__ void edges(const uint32_t* dst, const uint32_t*, const uint32_t*, const uint32_t*,
                                          const bool* valid) {
#pragma unroll
        for (int q = 0; q < kEdgesPerThread; ++q) {
            if (!valid[q]) continue;
            const uint32_t v = dst[q], wi = v >> 5, b = 1u << (v & 31);
            if (in_range(v, lo, hi)) {
                if (!(__ldcg(visited + wi) & b) && !(atomicOr(visited + wi, b) & b)) atomicOr(next + wi, b);
            } else if (mode == kDstRoute) {
                if (direct) {          // discovery in the owner's bitmaps over peer memory
                    const int q = route_owner(ro, v);
                    if (!(atomicOr(pw.vis[q] + wi, b) & b)) atomicOr(pw.nxt[q] + wi, b);
                } else if (!(__ldcg(sent + wi) & b) && !(atomicOr(sent + wi, b) & b)) {
                    route_push<uint32_t>(ro, v, v);
                }
            }
        }
    }
    __device__ void end_page() {}
};

// SSSP relaxation (kMin = dist) and WCC label propagation share one op: the
// payload of a selected vertex u is val[u]; an edge (u, v, w) offers val[u] + w
// (SSSP) or val[u] (WCC) to v, applied with atomicMin; an improvement marks v.
template <bool W, bool kSssp>
struct MMinOp {
    static constexpr bool kReadWeights = kSssp;
    static constexpr bool kWeighted = W;
    const uint32_t* cur;
    uint32_t* val;             // biased: val[v] for v in [lo, hi)
    uint32_t* next;
    unsigned long long nedges;
    bool ovf;
    uint32_t T;                // SSSP near-far threshold
    uint64_t lo, hi;
    int mode;
    RouteOut ro;
    int direct;                // GTS_ROUTE_PEER
    PeerWA pw;
    __device__ const uint32_t* frontier() const { return cur; }
    __device__ bool select(uint32_t v) { return test_bit(cur, v) && (!kSssp || __ldcg(val + v) <= T); }
    __device__ uint32_t payload(uint32_t v, uint32_t deg) {
        nedges += deg;
        return *((volatile uint32_t*)val + v);
    }
    __device__ bool select_lp(uint32_t vid, uint32_t, uint32_t len, uint32_t& pl) {
        if (!test_bit(cur, vid)) return false;
        pl = *((volatile uint32_t*)val + vid);
        if (kSssp && pl > T) return false;
        if (threadIdx.x == 0) nedges += len;
        return true;
    }
    __device__ __forceinline__ void edges(const uint32_t* dst, const uint32_t* w, const uint32_t* pu,
                                          const uint32_t*, const bool* valid) {
#pragma unroll
        for (int q = 0; q < kEdgesPerThread; ++q) {
            if (!valid[q]) continue;
            uint32_t cand = pu[q];
            if (kSssp) {
                const uint64_t nd = (uint64_t)pu[q] + w[q];
                if (nd >= (uint64_t)GTS_UNREACHED) {          // checked exactly after convergence
                    ovf = true;
                    continue;
                }
                cand = (uint32_t)nd;
            }
            const uint32_t v = dst[q];
            if (in_range(v, lo, hi)) {
                if (cand < __ldcg(val + v) && cand < atomicMin(val + v, cand)) atomicOr(next + (v >> 5), 1u << (v & 31));
            } else if (mode == kDstRoute) {
                if (direct) {          // atomicMin in the owner's WA over peer memory
                    const int q = route_owner(ro, v);
                    if (cand < atomicMin(pw.val[q] + v, cand)) atomicOr(pw.nxt[q] + (v >> 5), 1u << (v & 31));
                } else {
                    route_push<uint2>(ro, v, make_uint2(v, cand));
                }
            }
        }
    }
    __device__ void end_page() {}
};

template <bool W>
__global__ void __launch_bounds__(kThreads, 2)
mbfs_expand_kernel(PageSet ps, MBfsOp<W> op, uint32_t* work_ctr, unsigned long long* edges_out) {
    __shared__ TileSmem sm;
    expand_pages(ps, op, sm, work_ctr);
    block_add_u64(op.nedges, edges_out);
    if (op.direct) __threadfence_system();     // peer atomics before the kernel ends
}

template <bool W, bool kSssp>
__global__ void __launch_bounds__(kThreads, 2)
mmin_expand_kernel(PageSet ps, MMinOp<W, kSssp> op, uint32_t* work_ctr, unsigned long long* edges_out,
                   uint32_t* ovf_flag) {
    __shared__ TileSmem sm;
    expand_pages(ps, op, sm, work_ctr);
    block_add_u64(op.nedges, edges_out);
    if (__syncthreads_or(op.ovf) && threadIdx.x == 0) *ovf_flag = 1u;
    if (op.direct) __threadfence_system();
}

struct RecvView {
    const uint8_t* recv;
    uint64_t off[kMaxRanks];
    const unsigned long long* cnt;   // device, per peer
    int nranks;
};

// owner side of the routed BFS: exactly-once discovery of each received vertex
__global__ void bfs_apply_kernel(RecvView rv, uint32_t* visited, uint32_t* next) {
    const uint32_t* m = reinterpret_cast<const uint32_t*>(rv.recv);
    for (int p = 0; p < rv.nranks; ++p) {
        const uint64_t c = rv.cnt[p];
        for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < c; i += (uint64_t)gridDim.x * blockDim.x) {
            const uint32_t v = m[rv.off[p] + i], wi = v >> 5, b = 1u << (v & 31);
            if (!(atomicOr(visited + wi, b) & b)) atomicOr(next + wi, b);
        }
    }
}

// owner side of routed SSSP / WCC: val[v] = min(val[v], x), mark v if it decreased
__global__ void min_apply_kernel(RecvView rv, uint32_t* val, uint32_t* next) {
    const uint2* m = reinterpret_cast<const uint2*>(rv.recv);
    for (int p = 0; p < rv.nranks; ++p) {
        const uint64_t c = rv.cnt[p];
        for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < c; i += (uint64_t)gridDim.x * blockDim.x) {
            const uint2 e = m[rv.off[p] + i];
            if (e.y < atomicMin(val + e.x, e.y)) atomicOr(next + (e.x >> 5), 1u << (e.x & 31));
        }
    }
}

// val[v] = v and frontier bit set for every v in [lo, hi) (WCC label propagation start)
__global__ void wcc_lp_init_kernel(uint32_t* val, uint32_t* cur, uint64_t lo, uint64_t hi) {
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t v = lo + (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; v < hi; v += stride) {
        val[v] = (uint32_t)v;
        atomicOr(cur + (v >> 5), 1u << (v & 31));
    }
}

__global__ void set_source_range_kernel(uint32_t* value, uint32_t* visited, uint32_t* cur, uint64_t src) {
    value[src] = 0;
    if (visited) visited[src >> 5] |= 1u << (src & 31);
    cur[src >> 5] |= 1u << (src & 31);
}

struct MSlot {
    int r = 0;
    uint64_t lo = 0, hi = 0, w0 = 0, w1 = 0;   // WA range and the bitmap words it covers
    uint32_t *value = nullptr, *visited = nullptr, *cur = nullptr, *next = nullptr, *sent = nullptr;  // biased
    uint32_t *gathered = nullptr, *list = nullptr, *d_pages = nullptr;
    Counters* ctr = nullptr;
    uint32_t *cur0 = nullptr, *next0 = nullptr;   // the two frontier buffers as allocated (biased)
    std::array<uint32_t*, kMaxRanks> pval{}, pvis{}, pcur0{}, pnext0{};   // GTS_ROUTE_PEER: owners' WA
    std::vector<uint32_t> pages, h_list;
    Counters h = {};
};

constexpr int kBufMulti = 200;     // scratch slots of local slot i: kBufMulti + 16 i + k
constexpr int kBufRoute = 100;     // route buffers (comm.cu route_setup)
constexpr int kBufResult = 199;    // assembled full-n result

int traverse_multi(gts_context* c, const gts_graph* g, uint64_t src, const gts_run_config& rc, Ranks& R, void* out,
                   gts_run_stats* st, int algo, double t_start, bool streamed, double upload_s) {
    const uint64_t n = g->n, words = (n + 31) / 32;
    const int N = R.world, L = R.nloc;
    const uint32_t strat = rc.strategy;
    const bool route = strat == GTS_STRATEGY_S;
    // GTS_ROUTE_PEER: remote updates are atomics into the owner's WA over peer memory (the
    // expansion fused with the exchange); the owners' next bitmaps are double-buffered by level
    const bool peer = route && (rc.flags & GTS_ROUTE_PEER);
    const int mode = strat == GTS_STRATEGY_P ? kDstAll : route ? kDstRoute : kDstDrop;
    if (algo == kWCCLP && !route) return fail(GTS_EINVAL, "label propagation is the Strategy-S WCC");
    if (algo == kWCCLP && !g->symmetric)
        return fail(GTS_EUNSUPPORTED, "gts_wcc under Strategy-S needs pages built with GTS_BUILD_SYMMETRIC");
    const bool timing = rc.flags & GTS_RUN_TIMING;
    cudaStream_t s = c->stream;
    const int eg = c->num_sms * 4;
    std::vector<int32_t> owner;
    std::vector<uint64_t> vr;
    partition(g, strat, N, owner, vr);
    std::vector<MSlot> S(L);
    uint64_t wa_bytes = 0;
    for (int i = 0; i < L; ++i) {
        MSlot& m = S[i];
        m.r = R.rank(i);
        if (R.virt) {
            for (uint64_t j = 0; j < g->num_pages; ++j)
                if (strat == GTS_STRATEGY_S_BCAST || owner[j] == m.r) m.pages.push_back((uint32_t)j);
            GTS_TRY(c->buf(kBufMulti + 16 * i + 0, std::max<size_t>(m.pages.size(), 1) * 4, (void**)&m.d_pages));
            if (!m.pages.empty())
                GTS_CUDA(cudaMemcpyAsync(m.d_pages, m.pages.data(), m.pages.size() * 4, cudaMemcpyHostToDevice, s));
        } else {
            m.pages = c->dg.h_local_list;
            m.d_pages = c->dg.local_list;
        }
        if (strat == GTS_STRATEGY_P) {
            m.lo = 0;
            m.hi = n;
        } else {
            m.lo = vr[m.r];
            m.hi = vr[m.r + 1];
        }
        // WA: the full replicated arrays (P, S_BCAST) or this rank's range only (S)
        const uint64_t alo = route ? m.lo : 0, ahi = route ? m.hi : n;
        m.w0 = route ? alo >> 5 : 0;
        m.w1 = route ? (ahi + 31) >> 5 : words;
        const uint64_t nw = std::max<uint64_t>(m.w1 - m.w0, 1), nv = std::max<uint64_t>(ahi - alo, 1);
        uint32_t *val, *vis = nullptr, *cu, *nx;
        GTS_TRY(c->buf(kBufMulti + 16 * i + 1, nv * 4, (void**)&val));
        if (algo == kBFS) GTS_TRY(c->buf(kBufMulti + 16 * i + 2, nw * 4, (void**)&vis));
        GTS_TRY(c->buf(kBufMulti + 16 * i + 3, nw * 4, (void**)&cu));
        GTS_TRY(c->buf(kBufMulti + 16 * i + 4, nw * 4, (void**)&nx));
        m.value = val - alo;
        m.visited = vis ? vis - m.w0 : nullptr;
        m.cur = cu - m.w0;
        m.next = nx - m.w0;
        if (i == 0) wa_bytes = nv * 4 + nw * 4 * (algo == kBFS ? 3 : 2);
        if (!route) GTS_TRY(c->buf(kBufMulti + 16 * i + 5, (size_t)N * words * 4, (void**)&m.gathered));
        m.cur0 = m.cur;
        m.next0 = m.next;
        if (route && algo == kBFS && !peer) {
            GTS_TRY(c->buf(kBufMulti + 16 * i + 6, words * 4, (void**)&m.sent));
            GTS_CUDA(cudaMemsetAsync(m.sent, 0, words * 4, s));
            if (i == 0) wa_bytes += words * 4;
        }
        GTS_TRY(c->buf(kBufMulti + 16 * i + 7, std::max<uint64_t>(g->num_pages, 1) * 4, (void**)&m.list));
        GTS_TRY(c->buf(kBufMulti + 16 * i + 8, sizeof(Counters), (void**)&m.ctr));
        GTS_CUDA(cudaMemsetAsync(m.ctr, 0, sizeof(Counters), s));
        GTS_CUDA(cudaMemsetAsync(cu, 0, nw * 4, s));
        GTS_CUDA(cudaMemsetAsync(nx, 0, nw * 4, s));
        if (vis) GTS_CUDA(cudaMemsetAsync(vis, 0, nw * 4, s));
        if (algo == kWCCLP) {
            wcc_lp_init_kernel<<<eg, 256, 0, s>>>(m.value, m.cur, m.lo, m.hi);
            m.h_list = m.pages;            // every vertex starts active
        } else {
            GTS_CUDA(cudaMemsetAsync(val, 0xFF, nv * 4, s));
        }
    }
    const uint64_t isrc = algo == kWCCLP ? 0 : map_src(g, src);
    if (algo != kWCCLP) {
        // the pages holding src (Alg 1 line 5) among each rank's pages; its WA entry on its owner(s)
        auto it = std::upper_bound(g->start_vid.begin(), g->start_vid.end(), (uint32_t)isrc);
        const int64_t p = (int64_t)(it - g->start_vid.begin()) - 1;
        const int64_t a = g->kind[p] == GTS_PAGE_LP ? g->lp_first[p] : p, b = g->kind[p] == GTS_PAGE_LP ? g->lp_last[p] : p;
        for (MSlot& m : S) {
            for (int64_t q = a; q <= b; ++q)
                if (std::binary_search(m.pages.begin(), m.pages.end(), (uint32_t)q)) m.h_list.push_back((uint32_t)q);
            // the source's LV / dist and frontier bit: on its owner under S, in every replica
            // otherwise (P and S_BCAST keep the frontier and WA replicated)
            if (!route || (isrc >= m.lo && isrc < m.hi))
                set_source_range_kernel<<<1, 1, 0, s>>>(m.value, m.visited, m.cur, isrc);
        }
    }
    for (MSlot& m : S) {
        m.h.list_count = (uint32_t)m.h_list.size();
        if (!m.h_list.empty())
            GTS_CUDA(cudaMemcpyAsync(m.list, m.h_list.data(), m.h_list.size() * 4, cudaMemcpyHostToDevice, s));
        GTS_CUDA(cudaMemcpyAsync(&m.ctr->list_count, &m.h.list_count, 4, cudaMemcpyHostToDevice, s));
    }
    GTS_CUDA(cudaStreamSynchronize(s));        // host vectors above are read by the copies
    Route rt;
    if (peer) {                        // map every owner's WA allocations into this rank
        auto map = [&](auto get, auto put, bool words_bias) -> int {
            std::vector<void*> base(L);
            for (int i = 0; i < L; ++i) base[i] = get(S[i]);
            std::vector<std::array<void*, kMaxRanks>> pm;
            GTS_TRY(R.peer_map(base.data(), pm));
            for (int i = 0; i < L; ++i)
                for (int q = 0; q < N; ++q)
                    put(S[i], q, static_cast<uint32_t*>(pm[i][q]) - (words_bias ? (vr[q] >> 5) : vr[q]));
            return GTS_OK;
        };
        GTS_TRY(map([](MSlot& m) { return (void*)(m.value + m.lo); },
                    [](MSlot& m, int q, uint32_t* p) { m.pval[q] = p; }, false));
        if (algo == kBFS)
            GTS_TRY(map([](MSlot& m) { return (void*)(m.visited + m.w0); },
                        [](MSlot& m, int q, uint32_t* p) { m.pvis[q] = p; }, true));
        GTS_TRY(map([](MSlot& m) { return (void*)(m.cur0 + m.w0); },
                    [](MSlot& m, int q, uint32_t* p) { m.pcur0[q] = p; }, true));
        GTS_TRY(map([](MSlot& m) { return (void*)(m.next0 + m.w0); },
                    [](MSlot& m, int q, uint32_t* p) { m.pnext0[q] = p; }, true));
        GTS_TRY(R.barrier());          // every owner's WA is initialised before anyone writes into it
    } else if (route) {
        std::vector<std::vector<uint32_t>> pl(L);
        std::vector<const uint32_t*> dpl(L);
        for (int i = 0; i < L; ++i) {
            pl[i] = S[i].pages;
            dpl[i] = S[i].d_pages;
        }
        std::vector<std::array<uint64_t, kMaxRanks>> cap;
        GTS_TRY(route_capacities(c, g, R, rc, streamed, pl, dpl.data(), vr, 0, cap));
        GTS_TRY(route_setup(c, R, cap, algo == kBFS ? 4 : 8, kBufRoute, rt));
    }
    const uint64_t delta = rc.sssp_delta ? rc.sssp_delta : 0xFFFFFFFEull;
    uint32_t T = algo == kSSSP ? (uint32_t)std::min<uint64_t>(delta, 0xFFFFFFFEull) : 0xFFFFFFFEu;
    const bool W = g->weighted;
    const void* kexp = algo == kBFS ? (W ? (const void*)mbfs_expand_kernel<true> : (const void*)mbfs_expand_kernel<false>)
                       : algo == kSSSP ? (const void*)mmin_expand_kernel<true, true>
                                       : (W ? (const void*)mmin_expand_kernel<true, false>
                                            : (const void*)mmin_expand_kernel<false, false>);
    int grid = 0;
    GTS_TRY(sms_grid(c, kexp, kThreads, 0, &grid));
    uint64_t launches = 0, main_launches = 0, pages_processed = 0;
    uint32_t levels = 0;
    SweepStats ss;
    for (uint32_t lev = 0;; ++lev) {
        if (route && !peer) GTS_CUDA(cudaMemsetAsync(rt.d_scnt, 0, (size_t)L * kMaxRanks * 8, s));
        for (int i = 0; i < L; ++i) {
            MSlot& m = S[i];
            pages_processed += m.h.list_count;
            RouteOut ro{};
            if (route) {
                for (int q = 0; q <= N; ++q) ro.vr[q] = vr[q];
                ro.nranks = N;
            }
            if (route && !peer) {
                ro.send = rt.send[i];
                ro.cnt = rt.d_scnt + (size_t)i * kMaxRanks;
                ro.ovf = rt.d_ovf + i;
                for (int q = 0; q < N; ++q) {
                    ro.off[q] = rt.soff[i][q];
                    ro.cap[q] = rt.scap[i][q];
                }
            }
            PeerWA pwl{};
            if (peer)                  // this level's next bitmap of every owner: the buffers alternate
                for (int q = 0; q < N; ++q) {
                    pwl.val[q] = m.pval[q];
                    pwl.vis[q] = m.pvis[q];
                    pwl.nxt[q] = (lev & 1) ? m.pcur0[q] : m.pnext0[q];
                }
            auto launch = [&](const PageSet& ps, int gcap) -> int {
                GTS_CUDA(cudaMemsetAsync(&m.ctr->work, 0, 4, s));
                std::pair<cudaEvent_t, cudaEvent_t> ev;
                if (timing) { ev = c->t_main.next(); cudaEventRecord(ev.first, s); }
                PageSet p2 = ps;
                p2.split = 0u;
                const int gl = std::min(grid, gcap);
                if (algo == kBFS) {
                    if (W) {
                        MBfsOp<true> op{m.cur, m.visited, m.next, m.sent, 0ull, m.lo, m.hi, mode, ro, peer ? 1 : 0, pwl};
                        mbfs_expand_kernel<true><<<gl, kThreads, 0, s>>>(p2, op, &m.ctr->work, &m.ctr->edges);
                    } else {
                        MBfsOp<false> op{m.cur, m.visited, m.next, m.sent, 0ull, m.lo, m.hi, mode, ro, peer ? 1 : 0, pwl};
                        mbfs_expand_kernel<false><<<gl, kThreads, 0, s>>>(p2, op, &m.ctr->work, &m.ctr->edges);
                    }
                } else if (algo == kSSSP) {
                    MMinOp<true, true> op{m.cur, m.value, m.next, 0ull, false, T, m.lo, m.hi, mode, ro, peer ? 1 : 0, pwl};
                    mmin_expand_kernel<true, true><<<gl, kThreads, 0, s>>>(p2, op, &m.ctr->work, &m.ctr->edges,
                                                                         &m.ctr->flag);
                } else if (W) {
                    MMinOp<true, false> op{m.cur, m.value, m.next, 0ull, false, T, m.lo, m.hi, mode, ro, peer ? 1 : 0, pwl};
                    mmin_expand_kernel<true, false><<<gl, kThreads, 0, s>>>(p2, op, &m.ctr->work, &m.ctr->edges,
                                                                          &m.ctr->flag);
                } else {
                    MMinOp<false, false> op{m.cur, m.value, m.next, 0ull, false, T, m.lo, m.hi, mode, ro, peer ? 1 : 0, pwl};
                    mmin_expand_kernel<false, false><<<gl, kThreads, 0, s>>>(p2, op, &m.ctr->work, &m.ctr->edges,
                                                                           &m.ctr->flag);
                }
                if (timing) cudaEventRecord(ev.second, s);
                GTS_CUDA(cudaGetLastError());
                ++main_launches;
                return GTS_OK;
            };
            GTS_TRY(sweep_pages(c, g, rc, streamed, &m.h_list, m.list, m.h.list_count, &m.ctr->list_count, launch, &ss));
        }
        // ---- merge (a12) ----
        std::pair<cudaEvent_t, cudaEvent_t> ev;
        if (timing) { ev = c->t_merge.next(); cudaEventRecord(ev.first, s); }
        if (peer) {
            GTS_TRY(R.barrier());      // every rank's peer atomics of this level are done
        } else if (route) {
            GTS_TRY(R.route_exchange(rt));
            for (int i = 0; i < L; ++i) {
                RecvView rv{};
                rv.recv = rt.recv[i];
                for (int q = 0; q < N; ++q) rv.off[q] = rt.roff[i][q];
                rv.cnt = rt.d_rcnt + (size_t)i * kMaxRanks;
                rv.nranks = N;
                if (algo == kBFS) bfs_apply_kernel<<<eg, 256, 0, s>>>(rv, S[i].visited, S[i].next);
                else min_apply_kernel<<<eg, 256, 0, s>>>(rv, S[i].value, S[i].next);
                ++launches;
            }
        } else {
            if (algo == kSSSP) {           // dist: all-reduce(min) over the replicas
                std::vector<void*> b(L);
                for (int i = 0; i < L; ++i) b[i] = S[i].value;
                GTS_TRY(R.allreduce(b.data(), n, kCU32, kCMin));
            }
            std::vector<const void*> sb(L);
            std::vector<void*> rb(L);
            for (int i = 0; i < L; ++i) {
                sb[i] = S[i].next;
                rb[i] = S[i].gathered;
            }
            GTS_TRY(R.allgather(sb.data(), rb.data(), words * 4));
        }
        if (timing) { cudaEventRecord(ev.second, s); ev = c->t_finish.next(); cudaEventRecord(ev.first, s); }
        // ---- finish: merged next frontier, counts, next page set (a6) ----
        for (int i = 0; i < L; ++i) {
            MSlot& m = S[i];
            GTS_CUDA(cudaMemsetAsync(&m.ctr->count, 0, 8, s));
            GTS_CUDA(cudaMemsetAsync(&m.ctr->list_count, 0, 4, s));
            const uint32_t* gath = route ? nullptr : m.gathered;
            if (algo == kSSSP) {
                GTS_CUDA(cudaMemsetAsync(&m.ctr->near, 0, 8, s));
                GTS_CUDA(cudaMemsetAsync(&m.ctr->minpend, 0xFF, 4, s));
                sssp_finish_kernel<<<eg, 256, 0, s>>>(gath, N, words, m.w0, m.w1, m.cur, m.next, m.value, T,
                                                      &m.ctr->count, &m.ctr->near, &m.ctr->minpend);
            } else {
                frontier_finish_kernel<<<eg, 256, 0, s>>>(gath, N, words, m.w0, m.w1, m.next, m.visited,
                                                          algo == kBFS ? m.value : nullptr, lev + 1, &m.ctr->count);
            }
            frontier_pages_kernel<<<eg, 256, 0, s>>>(m.next, c->dg.rvt_start, c->dg.nslots, m.d_pages,
                                                     (uint32_t)m.pages.size(), m.list, &m.ctr->list_count);
            launches += 2;
            // GTS_ROUTE_PEER: this level's cur becomes the next level's next, which other ranks
            // write into once they pass the count all-reduce below -- clear it before it
            if (peer) GTS_CUDA(cudaMemsetAsync(m.cur + m.w0, 0, (m.w1 - m.w0) * 4, s));
        }
        if (route) {                       // frontier counts are per range: sum (SSSP: and min) over ranks
            std::vector<void*> b(L);
            for (int i = 0; i < L; ++i) b[i] = &S[i].ctr->count;
            GTS_TRY(R.allreduce(b.data(), 1, kCU64, kCSum));
            if (algo == kSSSP) {
                for (int i = 0; i < L; ++i) b[i] = &S[i].ctr->near;
                GTS_TRY(R.allreduce(b.data(), 1, kCU64, kCSum));
                for (int i = 0; i < L; ++i) b[i] = &S[i].ctr->minpend;
                GTS_TRY(R.allreduce(b.data(), 1, kCU32, kCMin));
            }
        }
        if (timing) cudaEventRecord(ev.second, s);
        GTS_CUDA(cudaGetLastError());
        for (MSlot& m : S) GTS_CUDA(cudaMemcpyAsync(&m.h, m.ctr, sizeof(Counters), cudaMemcpyDeviceToHost, s));
        GTS_CUDA(cudaStreamSynchronize(s));
        ++levels;
        if (S[0].h.count == 0) break;
        if (algo == kSSSP && S[0].h.near == 0) {
            const uint64_t nt = (uint64_t)S[0].h.minpend + delta;
            T = (uint32_t)std::min<uint64_t>(nt, 0xFFFFFFFEull);
        }
        for (MSlot& m : S) {
            if (streamed) {                // the host drives the copies: fetch and sort the page set
                m.h_list.resize(m.h.list_count);
                if (m.h.list_count) {
                    GTS_CUDA(cudaMemcpyAsync(m.h_list.data(), m.list, m.h.list_count * 4ull, cudaMemcpyDeviceToHost, s));
                    GTS_CUDA(cudaStreamSynchronize(s));
                    std::sort(m.h_list.begin(), m.h_list.end());
                    GTS_CUDA(cudaMemcpyAsync(m.list, m.h_list.data(), m.h.list_count * 4ull, cudaMemcpyHostToDevice, s));
                    GTS_CUDA(cudaStreamSynchronize(s));
                }
            }
            std::swap(m.cur, m.next);
            if (!peer) GTS_CUDA(cudaMemsetAsync(m.next + m.w0, 0, (m.w1 - m.w0) * 4, s));
        }
    }
    if (route && !peer) {
        bool ovf = false;
        GTS_TRY(R.route_overflow(rt, &ovf));
        if (ovf) return fail(GTS_ECUDA, "Strategy-S route region overflow (capacity count mismatch)");
    }
    // ---- result: every rank's range into one full array (a13) ----
    uint32_t* res = S[0].value;
    if (route) {
        GTS_TRY(c->buf(kBufResult, n * 4, (void**)&res));
        std::vector<void*> full(L, res);
        for (MSlot& m : S)
            if (m.hi > m.lo)
                GTS_CUDA(cudaMemcpyAsync(res + m.lo, m.value + m.lo, (m.hi - m.lo) * 4, cudaMemcpyDeviceToDevice, s));
        GTS_TRY(R.gather_ranges(full.data(), vr, 4));
    }
    if (algo == kSSSP) {                   // exact overflow test, on every rank, over its pages
        std::vector<void*> b(L);
        for (int i = 0; i < L; ++i) b[i] = &S[i].ctr->flag;
        GTS_TRY(R.allreduce(b.data(), 1, kCU32, kCMax));
        uint32_t flag = 0;
        GTS_CUDA(cudaMemcpyAsync(&flag, &S[0].ctr->flag, 4, cudaMemcpyDeviceToHost, s));
        GTS_CUDA(cudaStreamSynchronize(s));
        if (flag) {
            int g2 = 0;
            GTS_TRY(sms_grid(c, (const void*)sssp_check_kernel, kThreads, 0, &g2));
            for (int i = 0; i < L; ++i) {
                MSlot& m = S[i];
                GTS_CUDA(cudaMemsetAsync(&m.ctr->flag2, 0, 4, s));
                std::vector<uint32_t> hl = m.pages;
                GTS_TRY(sweep_pages(c, g, rc, streamed, &hl, m.d_pages, (uint32_t)hl.size(), nullptr,
                                    [&](const PageSet& ps, int gcap) -> int {
                                        GTS_CUDA(cudaMemsetAsync(&m.ctr->work, 0, 4, s));
                                        sssp_check_kernel<<<std::min(g2, gcap), kThreads, 0, s>>>(ps, res, &m.ctr->work,
                                                                                                &m.ctr->flag2);
                                        GTS_CUDA(cudaGetLastError());
                                        return GTS_OK;
                                    }, &ss));
            }
            for (int i = 0; i < L; ++i) b[i] = &S[i].ctr->flag2;
            GTS_TRY(R.allreduce(b.data(), 1, kCU32, kCMax));
            uint32_t bad = 0;
            GTS_CUDA(cudaMemcpyAsync(&bad, &S[0].ctr->flag2, 4, cudaMemcpyDeviceToHost, s));
            GTS_CUDA(cudaStreamSynchronize(s));
            if (bad) return fail(GTS_EOVERFLOW, "an SSSP distance reaches 2^32-1");
        }
    }
    GTS_TRY(deliver(c, g, res, out, rc.out_location, algo == kWCCLP));
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
        uint64_t edges = 0;
        for (MSlot& m : S) edges += m.h.edges;
        st->pages_processed = pages_processed;
        st->h2d_bytes = ss.h2d_bytes;
        st->edges_traversed = edges;
        st->nccl_bytes = R.bytes;
        st->launches = launches + main_launches;
        st->main_kernel_launches = main_launches;
        st->levels_or_iters = levels;
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

static int traverse(gts_context* c, const gts_graph* g, uint64_t src, const gts_run_config* cfg, uint32_t* out,
                    gts_run_stats* st, int algo) {
    clear_error();
    const double t_start = now_s();
    gts_run_config rc;
    GTS_TRY(validate_common(c, g, cfg, &rc));
    if (!out) return fail(GTS_EINVAL, "NULL output");
    if (src >= g->n) return fail(GTS_EINVAL, "src %llu >= n %llu", (unsigned long long)src, (unsigned long long)g->n);
    if (algo == kSSSP && !g->weighted) return fail(GTS_EUNSUPPORTED, "gts_sssp needs a graph built with weights");
    Ranks R;
    GTS_TRY(make_ranks(c, rc, &R));
    const uint64_t n = g->n, words = (n + 31) / 32;
    const uint64_t attr = R.world > 1 && rc.strategy == GTS_STRATEGY_S ? (4 * n + 16 * words) / R.world + words
                                                                         : 4 * n + 16 * words;
    const bool streamed = choose_streamed(c, g, rc, attr);
    double upload_s = 0;
    GTS_TRY(ensure_graph(c, g, rc.strategy, !streamed, &upload_s));
    if (R.world == 1) return traverse_single(c, g, src, rc, out, st, algo, t_start, streamed, upload_s);
    return traverse_multi(c, g, src, rc, R, out, st, algo, t_start, streamed, upload_s);
}

// ------------------------------------------------------------------- BC ---
// Betweenness centrality (Brandes) over the same page engine; the paper runs
// BC as a BFS-like algorithm on GTS (Fig 13c) without giving kernels.
// Per source: level by level, pass A is the BFS expansion (bfs_expand_kernel)
// and pass B adds sigma[u] into sigma[w] for every edge u->w from the level's
// frontier into the vertices discovered by pass A; then, over the stored level
// bitmaps in reverse, delta[v] += sigma[v]/sigma[w] * (1 + delta[w]) for every
// edge v->w with LV[w] = LV[v] + 1, each thread folding runs of the same source
// v before one fp64 atomic; finally bc[v] += delta[v] (v != source).

template <bool W>
struct BcSigmaOp {
    static constexpr bool kReadWeights = false;
    static constexpr bool kWeighted = W;
    const uint32_t* cur;
    const uint32_t* next;
    double* sigma;
    __device__ const uint32_t* frontier() const { return cur; }
    __device__ bool select(uint32_t v) { return test_bit(cur, v); }
    __device__ uint32_t payload(uint32_t, uint32_t) { return 0u; }
    __device__ bool select_lp(uint32_t vid, uint32_t, uint32_t, uint32_t&) { return test_bit(cur, vid); }
    __device__ __forceinline__ void edges(const uint32_t* dst, const uint32_t*, const uint32_t*, const uint32_t* src,
                                          const bool* ok) {
#pragma unroll
        for (int q = 0; q < kEdgesPerThread; ++q)
            if (ok[q] && test_bit(next, dst[q])) atomicAdd(sigma + dst[q], __ldcg(sigma + src[q]));
    }
    __device__ void end_page() {}
};

template <bool W>
struct BcDeltaOp {
    static constexpr bool kReadWeights = false;
    static constexpr bool kWeighted = W;
    const uint32_t* lvbits;    // vertices at level L
    const uint32_t* lv;
    uint32_t L;
    const double* sigma;
    double* delta;
    uint32_t run_src;
    double run_sum;
    bool has;
    __device__ const uint32_t* frontier() const { return lvbits; }
    __device__ bool select(uint32_t v) { return test_bit(lvbits, v); }
    __device__ uint32_t payload(uint32_t, uint32_t) { return 0u; }
    __device__ bool select_lp(uint32_t vid, uint32_t, uint32_t, uint32_t&) { return test_bit(lvbits, vid); }
    __device__ __forceinline__ void flush() {
        if (has && run_sum != 0.0) atomicAdd(delta + run_src, run_sum);
        has = false;
        run_sum = 0.0;
    }
    __device__ __forceinline__ void edges(const uint32_t* dst, const uint32_t*, const uint32_t*, const uint32_t* src,
                                          const bool* ok) {
        uint32_t l[kEdgesPerThread];
#pragma unroll
        for (int q = 0; q < kEdgesPerThread; ++q) l[q] = ok[q] ? __ldg(lv + dst[q]) : 0u;
#pragma unroll
        for (int q = 0; q < kEdgesPerThread; ++q) {
            if (!ok[q] || l[q] != L + 1) continue;
            const double cw = __ldg(sigma + src[q]) / __ldg(sigma + dst[q]) * (1.0 + __ldcg(delta + dst[q]));
            if (!has || run_src != src[q]) {
                flush();
                run_src = src[q];
                has = true;
            }
            run_sum += cw;
        }
    }
    __device__ void end_page() { flush(); }
};

template <bool W>
__global__ void __launch_bounds__(kThreads, 2)
bc_sigma_kernel(PageSet ps, const uint32_t* __restrict__ cur, const uint32_t* __restrict__ next, double* sigma,
                uint32_t* work_ctr) {
    __shared__ TileSmem sm;
    BcSigmaOp<W> op{cur, next, sigma};
    expand_pages(ps, op, sm, work_ctr);
}

template <bool W>
__global__ void __launch_bounds__(kThreads, 2)
bc_delta_kernel(PageSet ps, const uint32_t* __restrict__ lvbits, const uint32_t* __restrict__ lv, uint32_t L,
                const double* __restrict__ sigma, double* delta, uint32_t* work_ctr) {
    __shared__ TileSmem sm;
    BcDeltaOp<W> op{lvbits, lv, L, sigma, delta, 0u, 0.0, false};
    expand_pages(ps, op, sm, work_ctr);
    op.flush();
}

__global__ void bc_source_kernel(uint32_t* lv, uint32_t* visited, uint32_t* cur, double* sigma, uint64_t s) {
    lv[s] = 0;
    visited[s >> 5] |= 1u << (s & 31);
    cur[s >> 5] |= 1u << (s & 31);
    sigma[s] = 1.0;
}

__global__ void bc_accumulate_kernel(double* bc, const double* __restrict__ delta, uint64_t n, uint64_t s) {
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t v = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride)
        if (v != s) bc[v] += delta[v];
}

__global__ void gather_f64_kernel(double* out, const double* __restrict__ vals, const uint32_t* __restrict__ idx,
                                  uint64_t n) {
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t v = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride) out[v] = vals[idx[v]];
}

enum { kBufBcSigma = 40, kBufBcDelta, kBufBcOut, kBufBcList2, kBufBcTmp };

static int betweenness(gts_context* c, const gts_graph* g, const uint64_t* sources, uint32_t k,
                       const gts_run_config* cfg, double* out, gts_run_stats* st) {
    clear_error();
    const double t_start = now_s();
    gts_run_config rc;
    GTS_TRY(validate_common(c, g, cfg, &rc));
    if (!out || (k > 0 && !sources)) return fail(GTS_EINVAL, "NULL argument");
    for (uint32_t i = 0; i < k; ++i)
        if (sources[i] >= g->n) return fail(GTS_EINVAL, "source %llu >= n", (unsigned long long)sources[i]);
    if (c->world > 1) return fail(GTS_EUNSUPPORTED, "gts_bc runs on one GPU in this version");
    if (rc.flags & GTS_MICRO_MASK) return fail(GTS_EUNSUPPORTED, "GTS_MICRO_* techniques apply to gts_bfs and gts_pagerank");
    const uint64_t n = g->n, words = (n + 31) / 32;
    const bool streamed = choose_streamed(c, g, rc, 28 * n + 16 * words);
    double upload_s = 0;
    GTS_TRY(ensure_graph(c, g, rc.strategy, !streamed, &upload_s));
    const bool timing = rc.flags & GTS_RUN_TIMING;
    uint32_t *lv, *visited, *cur, *next, *list, *list2;
    double *sigma, *delta, *bc;
    Counters* ctr;
    GTS_TRY(c->buf(kBufValue, n * 4, (void**)&lv));
    GTS_TRY(c->buf(kBufVisited, words * 4, (void**)&visited));
    GTS_TRY(c->buf(kBufCur, words * 4, (void**)&cur));
    GTS_TRY(c->buf(kBufNext, words * 4, (void**)&next));
    GTS_TRY(c->buf(kBufList, std::max<uint64_t>(g->num_pages, 1) * 4, (void**)&list));
    GTS_TRY(c->buf(kBufBcList2, std::max<uint64_t>(g->num_pages, 1) * 4, (void**)&list2));
    GTS_TRY(c->buf(kBufCtr, sizeof(Counters), (void**)&ctr));
    GTS_TRY(c->buf(kBufBcSigma, n * 8, (void**)&sigma));
    GTS_TRY(c->buf(kBufBcDelta, n * 8, (void**)&delta));
    GTS_TRY(c->buf(kBufBcOut, n * 8, (void**)&bc));
    cudaStream_t s = c->stream;
    const int eg = c->num_sms * 4;
    GTS_CUDA(cudaMemsetAsync(bc, 0, n * 8, s));
    const bool wgt = g->weighted;
    const void* kA = wgt ? (const void*)bfs_expand_kernel<true> : (const void*)bfs_expand_kernel<false>;
    int grid = 0;
    GTS_TRY(sms_grid(c, kA, kThreads, 0, &grid));
    uint64_t launches = 1, main_launches = 0, pages_processed = 0, edges = 0;
    uint32_t levels_total = 0;
    SweepStats ss;
    uint32_t* lv_store = nullptr;             // per-level frontier bitmaps [lv_cap][words]
    uint32_t lv_cap = 0;
    struct Free { uint32_t*& p; ~Free() { cudaFree(p); } } free_store{lv_store};
    Counters h;
    for (uint32_t si = 0; si < k; ++si) {
        const uint64_t src = map_src(g, sources[si]);
        GTS_CUDA(cudaMemsetAsync(lv, 0xFF, n * 4, s));
        GTS_CUDA(cudaMemsetAsync(visited, 0, words * 4, s));
        GTS_CUDA(cudaMemsetAsync(cur, 0, words * 4, s));
        GTS_CUDA(cudaMemsetAsync(next, 0, words * 4, s));
        GTS_CUDA(cudaMemsetAsync(sigma, 0, n * 8, s));
        GTS_CUDA(cudaMemsetAsync(delta, 0, n * 8, s));
        GTS_CUDA(cudaMemsetAsync(ctr, 0, sizeof(Counters), s));
        bc_source_kernel<<<1, 1, 0, s>>>(lv, visited, cur, sigma, src);
        std::vector<uint32_t> l0 = pages_of_vertex(g, c->dg, c->rank, src);
        uint32_t* hs = (uint32_t*)c->h_small;
        hs[0] = (uint32_t)l0.size();
        if (!l0.empty()) GTS_CUDA(cudaMemcpyAsync(list, l0.data(), l0.size() * 4, cudaMemcpyHostToDevice, s));
        GTS_CUDA(cudaMemcpyAsync(&ctr->list_count, hs, 4, cudaMemcpyHostToDevice, s));
        std::vector<uint32_t> h_list = l0;
        uint32_t cur_count = (uint32_t)l0.size();
        std::vector<std::vector<uint32_t>> lvl_pages;  // streamed: page sets per level
        uint32_t L = 0;
        for (;; ++L) {
            // keep this level's frontier bitmap for the backward pass (the store grows
            // by doubling; earlier levels are copied over)
            if (L >= lv_cap) {
                const uint32_t ncap = std::max<uint32_t>(16, 2 * lv_cap);
                uint32_t* nb = nullptr;
                cudaError_t e = cudaMalloc(&nb, (size_t)ncap * words * 4);
                if (e != cudaSuccess) {
                    cudaGetLastError();
                    return fail(GTS_ENOMEM, "bc level bitmaps: cudaMalloc failed");
                }
                if (lv_store) {
                    GTS_CUDA(cudaMemcpyAsync(nb, lv_store, (size_t)lv_cap * words * 4, cudaMemcpyDeviceToDevice, s));
                    GTS_CUDA(cudaStreamSynchronize(s));
                    cudaFree(lv_store);
                }
                lv_store = nb;
                lv_cap = ncap;
            }
            GTS_CUDA(cudaMemcpyAsync(lv_store + (size_t)L * words, cur, words * 4, cudaMemcpyDeviceToDevice, s));
            if (streamed) lvl_pages.push_back(h_list);
            // pass A: discover level L+1 (BFS expansion)
            auto launchA = [&](const PageSet& ps, int cap) -> int {
                GTS_CUDA(cudaMemsetAsync(&ctr->work, 0, 4, s));
                std::pair<cudaEvent_t, cudaEvent_t> ev;
                if (timing) { ev = c->t_main.next(); cudaEventRecord(ev.first, s); }
                if (wgt) bfs_expand_kernel<true><<<std::min(grid, cap), kThreads, 0, s>>>(ps, cur, visited, next, &ctr->work, &ctr->edges, &ctr->vprefix_words, n, nullptr, 8u, 0xFFFFFFFFu);
                else bfs_expand_kernel<false><<<std::min(grid, cap), kThreads, 0, s>>>(ps, cur, visited, next, &ctr->work, &ctr->edges, &ctr->vprefix_words, n, nullptr, 8u, 0xFFFFFFFFu);
                if (timing) cudaEventRecord(ev.second, s);
                GTS_CUDA(cudaGetLastError());
                ++main_launches;
                return GTS_OK;
            };
            GTS_TRY(sweep_pages(c, g, rc, streamed, &h_list, list, cur_count, &ctr->list_count, launchA, &ss));
            GTS_CUDA(cudaMemsetAsync(&ctr->count, 0, 8, s));
            frontier_finish_kernel<<<eg, 256, 0, s>>>(nullptr, 1, words, 0, words, next, visited, lv, L + 1,
                                                      &ctr->count);
            // pass B: sigma of the newly discovered vertices
            auto launchB = [&](const PageSet& ps, int cap) -> int {
                GTS_CUDA(cudaMemsetAsync(&ctr->work, 0, 4, s));
                std::pair<cudaEvent_t, cudaEvent_t> ev;
                if (timing) { ev = c->t_main.next(); cudaEventRecord(ev.first, s); }
                if (wgt) bc_sigma_kernel<true><<<std::min(grid, cap), kThreads, 0, s>>>(ps, cur, next, sigma, &ctr->work);
                else bc_sigma_kernel<false><<<std::min(grid, cap), kThreads, 0, s>>>(ps, cur, next, sigma, &ctr->work);
                if (timing) cudaEventRecord(ev.second, s);
                GTS_CUDA(cudaGetLastError());
                ++main_launches;
                return GTS_OK;
            };
            GTS_TRY(sweep_pages(c, g, rc, streamed, &h_list, list, cur_count, &ctr->list_count, launchB, &ss));
            // next page set
            GTS_CUDA(cudaMemsetAsync(&ctr->list_count, 0, 4, s));
            frontier_pages_kernel<<<eg, 256, 0, s>>>(next, c->dg.rvt_start, c->dg.nslots, nullptr,
                                                     (uint32_t)g->num_pages, list, &ctr->list_count);
            launches += 3;
            GTS_CUDA(cudaMemcpyAsync(&h, ctr, sizeof(Counters), cudaMemcpyDeviceToHost, s));
            GTS_CUDA(cudaStreamSynchronize(s));
            pages_processed += 2ull * cur_count;
            if (h.count == 0) break;
            cur_count = h.list_count;
            if (streamed) {
                h_list.resize(h.list_count);
                GTS_CUDA(cudaMemcpyAsync(h_list.data(), list, h.list_count * 4ull, cudaMemcpyDeviceToHost, s));
                GTS_CUDA(cudaStreamSynchronize(s));
                std::sort(h_list.begin(), h_list.end());
                GTS_CUDA(cudaMemcpyAsync(list, h_list.data(), h.list_count * 4ull, cudaMemcpyHostToDevice, s));
            }
            std::swap(cur, next);
            GTS_CUDA(cudaMemsetAsync(next, 0, words * 4, s));
        }
        edges += h.edges;
        levels_total += L + 1;
        // backward: levels L-1 .. 0 (level L has no successors)
        for (int64_t q = (int64_t)L - 1; q >= 0; --q) {
            uint32_t* bits = lv_store + (size_t)q * words;
            GTS_CUDA(cudaMemsetAsync(&ctr->list_count, 0, 4, s));
            frontier_pages_kernel<<<eg, 256, 0, s>>>(bits, c->dg.rvt_start, c->dg.nslots, nullptr,
                                                     (uint32_t)g->num_pages, list2, &ctr->list_count);
            std::vector<uint32_t> hl;
            uint32_t cnt = 0;
            if (streamed) {
                hl = lvl_pages[q];
                cnt = (uint32_t)hl.size();
                GTS_CUDA(cudaMemcpyAsync(list2, hl.data(), hl.size() * 4, cudaMemcpyHostToDevice, s));
            }
            const uint32_t Lq = (uint32_t)q;
            auto launchD = [&](const PageSet& ps, int cap) -> int {
                GTS_CUDA(cudaMemsetAsync(&ctr->work, 0, 4, s));
                std::pair<cudaEvent_t, cudaEvent_t> ev;
                if (timing) { ev = c->t_main.next(); cudaEventRecord(ev.first, s); }
                if (wgt) bc_delta_kernel<true><<<std::min(grid, cap), kThreads, 0, s>>>(ps, bits, lv, Lq, sigma, delta, &ctr->work);
                else bc_delta_kernel<false><<<std::min(grid, cap), kThreads, 0, s>>>(ps, bits, lv, Lq, sigma, delta, &ctr->work);
                if (timing) cudaEventRecord(ev.second, s);
                GTS_CUDA(cudaGetLastError());
                ++main_launches;
                return GTS_OK;
            };
            GTS_TRY(sweep_pages(c, g, rc, streamed, &hl, list2, cnt, &ctr->list_count, launchD, &ss));
            ++launches;
        }
        bc_accumulate_kernel<<<eg, 256, 0, s>>>(bc, delta, n, src);
        ++launches;
    }
    // result in caller VIDs (fp64)
    if (g->ordered) {
        double* tmp;
        GTS_TRY(c->buf(kBufBcTmp, n * 8, (void**)&tmp));
        gather_f64_kernel<<<eg, 256, 0, s>>>(tmp, bc, c->dg.new_of_old, n);
        bc = tmp;
    }
    GTS_TRY(copy_out(c, bc, out, n * 8, rc.out_location));
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
        st->pages_processed = pages_processed;
        st->edges_traversed = edges;
        st->h2d_bytes = ss.h2d_bytes;
        st->launches = launches + main_launches;
        st->main_kernel_launches = main_launches;
        st->levels_or_iters = levels_total;
    } else if (timing) {
        c->t_main.sum_s();
        c->t_merge.sum_s();
        c->t_finish.sum_s();
        c->t_h2d.sum_s();
    }
    return GTS_OK;
}

}  // namespace gts

using namespace gts;

extern "C" int gts_bfs(gts_context* ctx, const gts_graph* g, uint64_t src, const gts_run_config* cfg,
                       uint32_t* level_out, gts_run_stats* stats) {
    return traverse(ctx, g, src, cfg, level_out, stats, kBFS);
}

extern "C" int gts_sssp(gts_context* ctx, const gts_graph* g, uint64_t src, const gts_run_config* cfg,
                        uint32_t* dist_out, gts_run_stats* stats) {
    return traverse(ctx, g, src, cfg, dist_out, stats, kSSSP);
}

extern "C" int gts_bc(gts_context* ctx, const gts_graph* g, const uint64_t* sources, uint32_t num_sources,
                      const gts_run_config* cfg, double* bc_out, gts_run_stats* stats) {
    return betweenness(ctx, g, sources, num_sources, cfg, bc_out, stats);
}
