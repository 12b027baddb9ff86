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

#include <cstring>

#include "expand.cuh"

namespace gts {

struct PrOp {
    static constexpr bool kReadWeights = false;
    const float* x;
    float* acc;
    float d;
    const uint32_t* hkeys;   // shared memory
    float* hacc;             // shared memory
    double dang;
    uint32_t last;
    float sum;
    bool has;

    __device__ bool select(uint32_t) { return true; }
    __device__ uint32_t payload(uint32_t v, uint32_t deg) {
        const float xv = __ldg(x + v);
        if (deg == 0) {
            dang += (double)xv;
            return 0u;
        }
        return __float_as_uint(d * xv / (float)deg);
    }
    __device__ bool select_lp(uint32_t vid, uint32_t total, uint32_t, uint32_t& pl) {
        pl = __float_as_uint(d * __ldg(x + vid) / (float)total);
        return true;
    }
    __device__ void emit(uint32_t dst, float c) {
        uint32_t b = hot_h1(dst);
        uint4 k = reinterpret_cast<const uint4*>(hkeys)[b];
        int way = k.x == dst ? 0 : k.y == dst ? 1 : k.z == dst ? 2 : k.w == dst ? 3 : -1;
        if (way < 0 && k.w != kHotEmpty) {              // h1 full: the key may sit in h2
            b = hot_h2(dst);
            k = reinterpret_cast<const uint4*>(hkeys)[b];
            way = k.x == dst ? 0 : k.y == dst ? 1 : k.z == dst ? 2 : k.w == dst ? 3 : -1;
        }
        if (way >= 0) atomicAdd(hacc + b * kHotWays + way, c);
        else atomicAdd(acc + dst, c);                   // RED.E.ADD.F32 (result unused)
    }
    __device__ void edge(uint32_t dst, uint32_t, uint32_t pl, uint32_t) {
        const float c = __uint_as_float(pl);
        if (has && dst == last) {
            sum += c;
            return;
        }
        if (has) emit(last, sum);
        last = dst;
        sum = c;
        has = true;
    }
    __device__ void end_page() {
        if (has) emit(last, sum);
        has = false;
    }
};

constexpr size_t kPrDynSmem = kHotSlots * (sizeof(uint32_t) + sizeof(float));

__global__ void __launch_bounds__(kThreads, 2)
pr_scatter_kernel(PageSet ps, const float* __restrict__ x, float* acc, const uint32_t* __restrict__ hot_keys,
                  float d, double* dang_out, uint32_t* work_ctr) {
    __shared__ TileSmem sm;
    extern __shared__ uint4 dyn_smem[];
    uint32_t* hkeys = reinterpret_cast<uint32_t*>(dyn_smem);
    float* hacc = reinterpret_cast<float*>(hkeys + kHotSlots);
    for (uint32_t i = threadIdx.x; i < kHotSlots; i += kThreads) {
        hkeys[i] = __ldg(hot_keys + i);
        hacc[i] = 0.f;
    }
    __syncthreads();
    PrOp op{x, acc, d, hkeys, hacc, 0.0, 0u, 0.f, false};
    expand_pages(ps, op, sm, work_ctr);
    __syncthreads();
    for (uint32_t i = threadIdx.x; i < kHotSlots; i += kThreads) {
        const uint32_t k = hkeys[i];
        const float v = hacc[i];
        if (k != kHotEmpty && v != 0.f) atomicAdd(acc + k, v);
    }
    double dg = op.dang;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) dg += __shfl_down_sync(0xFFFFFFFFu, dg, o);
    if ((threadIdx.x & 31) == 0 && dg != 0.0) atomicAdd(dang_out, dg);
}

__global__ void pr_init_kernel(float* x, float* acc, uint64_t n, float v0) {
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
        x[i] = v0;
        acc[i] = 0.f;
    }
}

// x_v <- (1-d)/n + d*D/n + acc_v ; acc_v <- 0  (float4 vectorised; buffers are 256-B aligned)
__global__ void pr_finish_kernel(float* x, float* acc, uint64_t n, double d, const double* dang, double* dang_reset,
                                 int uniform) {
    const double D = *dang;
    const float base = (float)((1.0 - d) / (double)n + (uniform ? d * D / (double)n : 0.0));
    const uint64_t n4 = n / 4;
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    float4* x4 = reinterpret_cast<float4*>(x);
    float4* a4 = reinterpret_cast<float4*>(acc);
    const float4 z = make_float4(0.f, 0.f, 0.f, 0.f);
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n4; i += stride) {
        float4 a = a4[i];
        x4[i] = make_float4(base + a.x, base + a.y, base + a.z, base + a.w);
        a4[i] = z;
    }
    for (uint64_t i = n4 * 4 + (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
        x[i] = base + acc[i];
        acc[i] = 0.f;
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) *dang_reset = 0.0;
}

enum { kBufX = 20, kBufAcc, kBufDang, kBufPrCtr };

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
    if (rc.residency == GTS_STREAMED) return fail(GTS_EUNSUPPORTED, "streamed residency not available for this call yet");
    if (rc.strategy == GTS_STRATEGY_S && c->world > 1) return fail(GTS_EUNSUPPORTED, "Strategy-S PageRank not available yet");
    double upload_s = 0;
    GTS_TRY(ensure_graph(c, g, rc.strategy, true, &upload_s));
    const bool timing = rc.flags & GTS_RUN_TIMING;
    const uint64_t n = g->n;
    float *x, *acc;
    double* dang;
    uint32_t* ctr;
    GTS_TRY(c->buf(kBufX, n * 4, (void**)&x));
    GTS_TRY(c->buf(kBufAcc, n * 4, (void**)&acc));
    GTS_TRY(c->buf(kBufDang, 2 * sizeof(double), (void**)&dang));
    GTS_TRY(c->buf(kBufPrCtr, 4, (void**)&ctr));
    cudaStream_t s = c->stream;
    static bool attr_set = false;
    if (!attr_set) {
        GTS_CUDA(cudaFuncSetAttribute(pr_scatter_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kPrDynSmem));
        attr_set = true;
    }
    int grid = 0;
    GTS_TRY(sms_grid(c, (const void*)pr_scatter_kernel, kThreads, kPrDynSmem, &grid));
    const int eg = c->num_sms * 4;
    pr_init_kernel<<<eg, 256, 0, s>>>(x, acc, n, (float)(1.0 / (double)n));
    GTS_CUDA(cudaMemsetAsync(dang, 0, 2 * sizeof(double), s));
    uint64_t launches = 1, main_launches = 0, nccl_bytes = 0;
    PageSet ps;
    ps.base = c->dg.pages;
    ps.list = c->dg.all_local ? nullptr : c->dg.local_list;
    ps.loc = c->dg.loc;
    ps.d_count = nullptr;
    ps.count = c->dg.n_local;
    ps.page_bytes = g->page_bytes;
    ps.mode = c->dg.all_local ? kAddrByPid : kAddrByLoc;
    ps.entry_encoding = g->entry_encoding;
    ps.rvt_start = c->dg.rvt_start;
    for (uint32_t it = 0; it < iters; ++it) {
        double* D = dang + (it & 1);
        GTS_CUDA(cudaMemsetAsync(ctr, 0, 4, s));
        std::pair<cudaEvent_t, cudaEvent_t> ev;
        if (timing) { ev = c->t_main.next(); cudaEventRecord(ev.first, s); }
        pr_scatter_kernel<<<grid, kThreads, kPrDynSmem, s>>>(ps, x, acc, c->dg.hot_keys, (float)damping, D, ctr);
        if (timing) cudaEventRecord(ev.second, s);
        GTS_CUDA(cudaGetLastError());
        ++launches;
        ++main_launches;
        if (c->world > 1) {
            if (timing) { ev = c->t_merge.next(); cudaEventRecord(ev.first, s); }
            GTS_NCCL(ncclGroupStart());
            GTS_NCCL(ncclAllReduce(acc, acc, n, ncclFloat32, ncclSum, c->comm, s));
            GTS_NCCL(ncclAllReduce(D, D, 1, ncclFloat64, ncclSum, c->comm, s));
            GTS_NCCL(ncclGroupEnd());
            if (timing) cudaEventRecord(ev.second, s);
            nccl_bytes += n * 4 + 8;
        }
        if (timing) { ev = c->t_finish.next(); cudaEventRecord(ev.first, s); }
        pr_finish_kernel<<<eg, 256, 0, s>>>(x, acc, n, damping, D, dang + ((it + 1) & 1),
                                             dangling == GTS_DANGLING_UNIFORM ? 1 : 0);
        if (timing) cudaEventRecord(ev.second, s);
        ++launches;
    }
    GTS_CUDA(cudaGetLastError());
    GTS_TRY(copy_out(c, x, rank_out, n * 4, rc.out_location));
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
        st->edges_traversed = g->m * (uint64_t)iters / (uint64_t)c->world;
        st->nccl_bytes = nccl_bytes;
        st->launches = launches;
        st->main_kernel_launches = main_launches;
        st->levels_or_iters = iters;
    } else if (timing) {
        c->t_main.sum_s();
        c->t_merge.sum_s();
        c->t_finish.sum_s();
    }
    return GTS_OK;
}
