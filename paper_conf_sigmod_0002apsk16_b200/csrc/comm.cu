// Ranks, merges and routed exchange; see comm.h.
//
// Real ranks: NCCL collectives on the context's communicator over NVLink
// (P:344-354 Strategy-P merges; P:430-440 Strategy-S).  NCCL has no bitwise
// OR, so BFS frontiers are all-gathered and OR-ed by the finish kernels.
// Virtual ranks: the same collectives over the V slots' device buffers, with
// device-to-device copies and reduction kernels on the compute stream.
#include <cuda_runtime.h>
#include <nccl.h>

#include <algorithm>
#include <cstring>

#include "comm.h"
#include "expand.cuh"
#include "sweep.cuh"

namespace gts {

struct PtrArr {
    void* p[kMaxRanks];
};

template <class T>
__device__ __forceinline__ T cop(T a, T b, int op) {
    return op == kCSum ? a + b : op == kCMin ? (b < a ? b : a) : (b > a ? b : a);
}

// bufs[0..V) element-wise reduced (in rank order) and written back to all.
template <class T>
__global__ void vr_allreduce_kernel(PtrArr bufs, int V, size_t count, int op) {
    const size_t stride = (size_t)gridDim.x * blockDim.x;
    for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < count; i += stride) {
        T a = reinterpret_cast<T*>(bufs.p[0])[i];
        for (int r = 1; r < V; ++r) a = cop(a, reinterpret_cast<T*>(bufs.p[r])[i], op);
        for (int r = 0; r < V; ++r) reinterpret_cast<T*>(bufs.p[r])[i] = a;
    }
}

// owner q's acc (biased, absolute index) += sum over ranks of part[rank][v], v in [a_q, b_q); parts zeroed
struct Ranges {
    uint64_t a[kMaxRanks], b[kMaxRanks];
};

__global__ void vr_reduce_owners_kernel(PtrArr part, PtrArr dst, Ranges rg, int V) {
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (int q = 0; q < V; ++q) {
        float* d = reinterpret_cast<float*>(dst.p[q]);
        for (uint64_t v = rg.a[q] + (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; v < rg.b[q]; v += stride) {
            float s = 0.f;
            for (int r = 0; r < V; ++r) {
                float* pr = reinterpret_cast<float*>(part.p[r]);
                s += pr[v];
                pr[v] = 0.f;
            }
            if (s != 0.f) d[v] += s;
        }
    }
}

// acc[v] += in[v], in[v] = 0 over [a, b) (acc biased: absolute index)
__global__ void add_range_kernel(float* acc, float* in, uint64_t a, uint64_t b) {
    for (uint64_t v = a + (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; v < b; v += (uint64_t)gridDim.x * blockDim.x) {
        const float x = in[v];
        if (x != 0.f) acc[v] += x;
        in[v] = 0.f;
    }
}

static ncclDataType_t nccl_type(CType t) {
    return t == kCF32 ? ncclFloat32 : t == kCF64 ? ncclFloat64 : t == kCU32 ? ncclUint32 : ncclUint64;
}
static ncclRedOp_t nccl_op(COp o) { return o == kCSum ? ncclSum : o == kCMin ? ncclMin : ncclMax; }
static size_t type_size(CType t) { return t == kCF32 || t == kCU32 ? 4 : 8; }

int make_ranks(Context* c, const gts_run_config& rc, Ranks* R) {
    R->c = c;
    R->bytes = 0;
    const uint32_t V = rc.virtual_ranks;
    if (c->world > 1) {
        if (V > 1) return fail(GTS_EINVAL, "virtual_ranks needs a world-1 context (this one has %d ranks)", c->world);
        if (c->world > kMaxRanks) return fail(GTS_EUNSUPPORTED, "at most %d ranks", kMaxRanks);
        R->world = c->world;
        R->r0 = c->rank;
        R->nloc = 1;
        R->virt = false;
    } else if (V > 1) {
        if (V > (uint32_t)kMaxRanks) return fail(GTS_EINVAL, "virtual_ranks must be <= %d", kMaxRanks);
        R->world = (int)V;
        R->r0 = 0;
        R->nloc = (int)V;
        R->virt = true;
    } else {
        R->world = 1;
        R->r0 = 0;
        R->nloc = 1;
        R->virt = false;
    }
    return GTS_OK;
}

int Ranks::allreduce(void* const* bufs, size_t count, CType t, COp op) {
    if (world == 1 || count == 0) return GTS_OK;
    cudaStream_t s = c->stream;
    bytes += count * type_size(t) * nloc;     // (bytes: summed over the ranks this process runs)
    if (!virt) {
        GTS_NCCL(ncclAllReduce(bufs[0], bufs[0], count, nccl_type(t), nccl_op(op), c->comm, s));
        return GTS_OK;
    }
    PtrArr pa{};
    for (int i = 0; i < nloc; ++i) pa.p[i] = bufs[i];
    const int grid = c->num_sms * 4;
    switch (t) {
        case kCF32: vr_allreduce_kernel<float><<<grid, 256, 0, s>>>(pa, nloc, count, op); break;
        case kCF64: vr_allreduce_kernel<double><<<grid, 256, 0, s>>>(pa, nloc, count, op); break;
        case kCU32: vr_allreduce_kernel<uint32_t><<<grid, 256, 0, s>>>(pa, nloc, count, op); break;
        case kCU64: vr_allreduce_kernel<unsigned long long><<<grid, 256, 0, s>>>(pa, nloc, count, op); break;
    }
    GTS_CUDA(cudaGetLastError());
    return GTS_OK;
}

int Ranks::allgather(const void* const* send, void* const* recv, size_t nbytes) {
    cudaStream_t s = c->stream;
    bytes += nbytes * nloc;
    if (!virt) {
        if (world == 1) {
            if (recv[0] != send[0]) GTS_CUDA(cudaMemcpyAsync(recv[0], send[0], nbytes, cudaMemcpyDeviceToDevice, s));
            return GTS_OK;
        }
        GTS_NCCL(ncclAllGather(send[0], recv[0], nbytes, ncclUint8, c->comm, s));
        return GTS_OK;
    }
    for (int i = 0; i < nloc; ++i)
        for (int r = 0; r < nloc; ++r)
            GTS_CUDA(cudaMemcpyAsync(static_cast<uint8_t*>(recv[i]) + (size_t)r * nbytes, send[r], nbytes,
                                     cudaMemcpyDeviceToDevice, s));
    return GTS_OK;
}

int Ranks::gather_ranges(void* const* full, const std::vector<uint64_t>& vr, size_t es) {
    if (world == 1) return GTS_OK;
    cudaStream_t s = c->stream;
    if (!virt) {
        GTS_NCCL(ncclGroupStart());
        for (int q = 0; q < world; ++q)
            if (vr[q + 1] > vr[q]) {
                uint8_t* p = static_cast<uint8_t*>(full[0]) + vr[q] * es;
                GTS_NCCL(ncclBroadcast(p, p, (vr[q + 1] - vr[q]) * es, ncclUint8, q, c->comm, s));
            }
        GTS_NCCL(ncclGroupEnd());
        bytes += (vr[r0 + 1] - vr[r0]) * es;
        return GTS_OK;
    }
    bytes += (vr[nloc] - vr[0]) * es;
    for (int i = 0; i < nloc; ++i)
        for (int q = 0; q < nloc; ++q)
            if (q != i && full[q] != full[i] && vr[q + 1] > vr[q])
                GTS_CUDA(cudaMemcpyAsync(static_cast<uint8_t*>(full[i]) + vr[q] * es,
                                         static_cast<uint8_t*>(full[q]) + vr[q] * es, (vr[q + 1] - vr[q]) * es,
                                         cudaMemcpyDeviceToDevice, s));
    return GTS_OK;
}

int Ranks::reduce_to_owners(float* const* part, float* const* dst, const std::vector<uint64_t>& vr, uint64_t limit) {
    cudaStream_t s = c->stream;
    const int grid = c->num_sms * 4;
    if (limit == 0) return GTS_OK;
    if (!virt) {
        // tmp (absolute index) receives the owner's slice of the summed partials
        float* tmp;
        GTS_TRY(c->buf(95, limit * 4, (void**)&tmp));
        GTS_NCCL(ncclGroupStart());
        for (int q = 0; q < world; ++q) {
            const uint64_t a = std::min<uint64_t>(vr[q], limit), b = std::min<uint64_t>(vr[q + 1], limit);
            if (b > a) GTS_NCCL(ncclReduce(part[0] + a, tmp + a, b - a, ncclFloat32, ncclSum, q, c->comm, s));
        }
        GTS_NCCL(ncclGroupEnd());
        bytes += limit * 4;
        const uint64_t a = std::min<uint64_t>(vr[r0], limit), b = std::min<uint64_t>(vr[r0 + 1], limit);
        if (b > a) add_range_kernel<<<grid, 256, 0, s>>>(dst[0], tmp, a, b);
        GTS_CUDA(cudaMemsetAsync(part[0], 0, limit * 4, s));
        GTS_CUDA(cudaGetLastError());
        return GTS_OK;
    }
    bytes += limit * 4 * nloc;
    PtrArr pp{}, pd{};
    Ranges rg{};
    for (int i = 0; i < nloc; ++i) {
        pp.p[i] = part[i];
        pd.p[i] = dst[i];
        rg.a[i] = std::min<uint64_t>(vr[i], limit);
        rg.b[i] = std::min<uint64_t>(vr[i + 1], limit);
    }
    vr_reduce_owners_kernel<<<grid, 256, 0, s>>>(pp, pd, rg, nloc);
    GTS_CUDA(cudaGetLastError());
    return GTS_OK;
}

int Ranks::route_exchange(Route& rt) {
    cudaStream_t s = c->stream;
    const int N = world;
    rt.h_rcnt.assign(nloc, {});
    if (!virt) {
        // counts, then payloads; self-messages never exist (local updates are applied in place)
        const int me = r0;
        unsigned long long* scnt = rt.d_scnt;
        unsigned long long* rcnt = rt.d_rcnt;
        GTS_NCCL(ncclGroupStart());
        for (int p = 0; p < N; ++p) {
            if (p == me) continue;
            GTS_NCCL(ncclSend(scnt + p, 1, ncclUint64, p, c->comm, s));
            GTS_NCCL(ncclRecv(rcnt + p, 1, ncclUint64, p, c->comm, s));
        }
        GTS_NCCL(ncclGroupEnd());
        std::array<unsigned long long, kMaxRanks> hs{}, hr{};
        GTS_CUDA(cudaMemcpyAsync(hs.data(), scnt, kMaxRanks * 8, cudaMemcpyDeviceToHost, s));
        GTS_CUDA(cudaMemcpyAsync(hr.data(), rcnt, kMaxRanks * 8, cudaMemcpyDeviceToHost, s));
        GTS_CUDA(cudaStreamSynchronize(s));
        // clamp to the capacities: a sender that overflowed wrote only cap messages (and raised
        // its flag, combined over ranks by route_overflow before anyone returns)
        GTS_NCCL(ncclGroupStart());
        for (int p = 0; p < N; ++p) {
            if (p == me) continue;
            const uint64_t sc = std::min<uint64_t>(hs[p], rt.scap[0][p]);
            const uint64_t rc = std::min<uint64_t>(hr[p], rt.rcap[0][p]);
            if (sc) GTS_NCCL(ncclSend(rt.send[0] + rt.soff[0][p] * rt.esize, sc * rt.esize, ncclUint8, p, c->comm, s));
            if (rc) GTS_NCCL(ncclRecv(rt.recv[0] + rt.roff[0][p] * rt.esize, rc * rt.esize, ncclUint8, p, c->comm, s));
            rt.h_rcnt[0][p] = rc;
            rt.sent_msgs += sc;
            bytes += sc * rt.esize;
        }
        GTS_NCCL(ncclGroupEnd());
        rt.h_rcnt[0][me] = 0;
        GTS_CUDA(cudaMemcpyAsync(rcnt, rt.h_rcnt[0].data(), kMaxRanks * 8, cudaMemcpyHostToDevice, s));
        GTS_CUDA(cudaStreamSynchronize(s));   // h_rcnt is host memory read by the copy
        return GTS_OK;
    }
    std::vector<unsigned long long> hs((size_t)nloc * kMaxRanks);
    GTS_CUDA(cudaMemcpyAsync(hs.data(), rt.d_scnt, hs.size() * 8, cudaMemcpyDeviceToHost, s));
    GTS_CUDA(cudaStreamSynchronize(s));
    for (int snd = 0; snd < nloc; ++snd)
        for (int p = 0; p < nloc; ++p) {
            if (p == snd) continue;
            const uint64_t cnt = std::min<uint64_t>(std::min<uint64_t>(hs[(size_t)snd * kMaxRanks + p], rt.scap[snd][p]),
                                                    rt.rcap[p][snd]);
            if (cnt)
                GTS_CUDA(cudaMemcpyAsync(rt.recv[p] + rt.roff[p][snd] * rt.esize, rt.send[snd] + rt.soff[snd][p] * rt.esize,
                                         cnt * rt.esize, cudaMemcpyDeviceToDevice, s));
            rt.h_rcnt[p][snd] = cnt;
            rt.sent_msgs += cnt;
            bytes += cnt * rt.esize;
        }
    std::vector<unsigned long long> hr((size_t)nloc * kMaxRanks, 0);
    for (int p = 0; p < nloc; ++p)
        for (int q = 0; q < kMaxRanks; ++q) hr[(size_t)p * kMaxRanks + q] = rt.h_rcnt[p][q];
    GTS_CUDA(cudaMemcpyAsync(rt.d_rcnt, hr.data(), hr.size() * 8, cudaMemcpyHostToDevice, s));
    GTS_CUDA(cudaStreamSynchronize(s));
    return GTS_OK;
}

int Ranks::route_overflow(Route& rt, bool* any) {
    std::vector<uint32_t> h(nloc, 0);
    void* bufs[kMaxRanks];
    for (int i = 0; i < nloc; ++i) bufs[i] = rt.d_ovf + i;
    GTS_TRY(allreduce(bufs, 1, kCU32, kCMax));
    GTS_CUDA(cudaMemcpyAsync(h.data(), rt.d_ovf, nloc * 4, cudaMemcpyDeviceToHost, c->stream));
    GTS_CUDA(cudaStreamSynchronize(c->stream));
    *any = false;
    for (uint32_t v : h) *any |= v != 0;
    return GTS_OK;
}

int Ranks::barrier() {
    if (world == 1 || virt) return GTS_OK;            // virtual ranks share one stream
    uint64_t* d;
    GTS_TRY(c->buf(98, 8, (void**)&d));
    GTS_NCCL(ncclAllReduce(d, d, 1, ncclUint64, ncclSum, c->comm, c->stream));
    return GTS_OK;
}

int Ranks::peer_map(void* const* base, std::vector<std::array<void*, kMaxRanks>>& out) {
    out.assign(nloc, {});
    if (virt || world == 1) {
        for (int i = 0; i < nloc; ++i)
            for (int q = 0; q < nloc; ++q) out[i][q] = base[q];
        return GTS_OK;
    }
    // real ranks: all-gather the IPC handles of every rank's allocation, open the peers'
    cudaIpcMemHandle_t mine;
    GTS_CUDA(cudaIpcGetMemHandle(&mine, base[0]));
    uint8_t* d;
    GTS_TRY(c->buf(99, sizeof(cudaIpcMemHandle_t) * (world + 1), (void**)&d));
    GTS_CUDA(cudaMemcpyAsync(d, &mine, sizeof(mine), cudaMemcpyHostToDevice, c->stream));
    GTS_NCCL(ncclAllGather(d, d + sizeof(mine), sizeof(mine), ncclUint8, c->comm, c->stream));
    std::vector<cudaIpcMemHandle_t> all(world);
    GTS_CUDA(cudaMemcpyAsync(all.data(), d + sizeof(mine), sizeof(mine) * world, cudaMemcpyDeviceToHost, c->stream));
    GTS_CUDA(cudaStreamSynchronize(c->stream));
    for (int q = 0; q < world; ++q) {
        if (q == r0) {
            out[0][q] = base[0];
            continue;
        }
        const std::string key(reinterpret_cast<const char*>(&all[q]), sizeof(cudaIpcMemHandle_t));
        auto it = c->ipc_open.find(key);
        if (it == c->ipc_open.end()) {
            void* p = nullptr;
            GTS_CUDA(cudaIpcOpenMemHandle(&p, all[q], cudaIpcMemLazyEnablePeerAccess));
            it = c->ipc_open.emplace(key, p).first;
        }
        out[0][q] = it->second;
    }
    return GTS_OK;
}

// ---- capacities: remote edges per (sender, owner) --------------------------

template <bool W>
struct RouteCountOp {
    static constexpr bool kReadWeights = false;
    static constexpr bool kWeighted = W;
    uint64_t vr[kMaxRanks + 1];
    int nranks, me;
    uint32_t skip_below;
    unsigned long long cnt[kMaxRanks];
    __device__ const uint32_t* frontier() const { return nullptr; }
    __device__ bool select(uint32_t) { return true; }
    __device__ uint32_t payload(uint32_t, uint32_t) { return 0u; }
    __device__ bool select_lp(uint32_t, uint32_t, uint32_t, uint32_t&) { return true; }
    __device__ __forceinline__ void edges(const uint32_t* dst, const uint32_t*, const uint32_t*, const uint32_t*,
                                          const bool* ok) {
#pragma unroll
        for (int q = 0; q < kEdgesPerThread; ++q) {
            const uint32_t v = dst[q];
            if (!ok[q] || v < skip_below) continue;
            int p = 0;
            while (p < nranks - 1 && (uint64_t)v >= vr[p + 1]) ++p;
            if (p == me) continue;
#pragma unroll
            for (int k = 0; k < kMaxRanks; ++k) cnt[k] += (k == p);
        }
    }
    __device__ void end_page() {}
};

template <bool W>
__global__ void __launch_bounds__(kThreads, 2)
route_count_kernel(PageSet ps, RouteCountOp<W> op, unsigned long long* out, uint32_t* work_ctr) {
    __shared__ TileSmem sm;
    expand_pages(ps, op, sm, work_ctr);
#pragma unroll
    for (int k = 0; k < kMaxRanks; ++k) {
        unsigned long long v = op.cnt[k];
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) v += __shfl_down_sync(0xFFFFFFFFu, v, o);
        if ((threadIdx.x & 31) == 0 && v) atomicAdd(out + k, v);
    }
}

int route_capacities(Context* c, const Graph* g, Ranks& R, const gts_run_config& rc, bool streamed,
                     const std::vector<std::vector<uint32_t>>& plist, const uint32_t* const* d_plist,
                     const std::vector<uint64_t>& vr, uint32_t skip_below,
                     std::vector<std::array<uint64_t, kMaxRanks>>& cap) {
    const int N = R.world;
    DevGraph& dg = c->dg;
    const uint64_t key = ((uint64_t)skip_below << 8) ^ ((uint64_t)N << 1) ^ (R.virt ? 1 : 0) ^
                         ((uint64_t)rc.strategy << 60);
    cap.assign(N, {});
    auto it = dg.route_caps.find(key);
    if (it != dg.route_caps.end()) {
        for (int r = 0; r < N; ++r)
            for (int p = 0; p < kMaxRanks; ++p) cap[r][p] = it->second[(size_t)r * kMaxRanks + p];
        return GTS_OK;
    }
    cudaStream_t s = c->stream;
    unsigned long long* d_cnt;
    uint32_t* ctr;
    GTS_TRY(c->buf(96, (size_t)R.nloc * kMaxRanks * 8 + 16, (void**)&d_cnt));
    ctr = reinterpret_cast<uint32_t*>(d_cnt + (size_t)R.nloc * kMaxRanks);
    GTS_CUDA(cudaMemsetAsync(d_cnt, 0, (size_t)R.nloc * kMaxRanks * 8, s));
    const void* k = g->weighted ? (const void*)route_count_kernel<true> : (const void*)route_count_kernel<false>;
    int grid = 0;
    GTS_TRY(sms_grid(c, k, kThreads, 0, &grid));
    SweepStats ss;
    for (int i = 0; i < R.nloc; ++i) {
        const int r = R.rank(i);
        std::vector<uint32_t> hl(plist[i]);
        GTS_TRY(sweep_pages(c, g, rc, streamed, &hl, d_plist[i], (uint32_t)hl.size(), nullptr,
                            [&](const PageSet& ps, int gcap) -> int {
                                GTS_CUDA(cudaMemsetAsync(ctr, 0, 4, s));
                                unsigned long long* out = d_cnt + (size_t)i * kMaxRanks;
                                if (g->weighted) {
                                    RouteCountOp<true> op{};
                                    for (int q = 0; q <= N; ++q) op.vr[q] = vr[q];
                                    op.nranks = N;
                                    op.me = r;
                                    op.skip_below = skip_below;
                                    route_count_kernel<true><<<std::min(grid, gcap), kThreads, 0, s>>>(ps, op, out, ctr);
                                } else {
                                    RouteCountOp<false> op{};
                                    for (int q = 0; q <= N; ++q) op.vr[q] = vr[q];
                                    op.nranks = N;
                                    op.me = r;
                                    op.skip_below = skip_below;
                                    route_count_kernel<false><<<std::min(grid, gcap), kThreads, 0, s>>>(ps, op, out, ctr);
                                }
                                GTS_CUDA(cudaGetLastError());
                                return GTS_OK;
                            }, &ss));
    }
    std::vector<unsigned long long> h((size_t)N * kMaxRanks, 0);
    if (R.virt || N == 1) {
        GTS_CUDA(cudaMemcpyAsync(h.data(), d_cnt, (size_t)R.nloc * kMaxRanks * 8, cudaMemcpyDeviceToHost, s));
    } else {   // every rank learns every sender's row (receivers size their regions from it)
        unsigned long long* all;
        GTS_TRY(c->buf(97, (size_t)N * kMaxRanks * 8, (void**)&all));
        GTS_NCCL(ncclAllGather(d_cnt, all, kMaxRanks, ncclUint64, c->comm, s));
        GTS_CUDA(cudaMemcpyAsync(h.data(), all, (size_t)N * kMaxRanks * 8, cudaMemcpyDeviceToHost, s));
    }
    GTS_CUDA(cudaStreamSynchronize(s));
    std::vector<uint64_t> flat(h.begin(), h.end());
    for (int r = 0; r < N; ++r)
        for (int p = 0; p < kMaxRanks; ++p) cap[r][p] = flat[(size_t)r * kMaxRanks + p];
    dg.route_caps[key] = std::move(flat);
    return GTS_OK;
}

int route_setup(Context* c, Ranks& R, const std::vector<std::array<uint64_t, kMaxRanks>>& cap, size_t esize, int base,
                Route& rt) {
    const int N = R.world, L = R.nloc;
    rt.esize = esize;
    rt.send.assign(L, nullptr);
    rt.recv.assign(L, nullptr);
    rt.soff.assign(L, {});
    rt.scap.assign(L, {});
    rt.roff.assign(L, {});
    rt.rcap.assign(L, {});
    rt.sent_msgs = 0;
    for (int i = 0; i < L; ++i) {
        const int r = R.rank(i);
        uint64_t st = 0, rt_ = 0;
        for (int p = 0; p < N; ++p) {
            rt.soff[i][p] = st;
            rt.scap[i][p] = p == r ? 0 : cap[r][p];
            st += rt.scap[i][p];
            rt.roff[i][p] = rt_;
            rt.rcap[i][p] = p == r ? 0 : cap[p][r];
            rt_ += rt.rcap[i][p];
        }
        GTS_TRY(c->buf(base + i, std::max<uint64_t>(st, 1) * esize, (void**)&rt.send[i]));
        GTS_TRY(c->buf(base + L + i, std::max<uint64_t>(rt_, 1) * esize, (void**)&rt.recv[i]));
    }
    uint8_t* meta;
    const size_t cb = (size_t)L * kMaxRanks * 8;
    GTS_TRY(c->buf(base + 2 * L, 2 * cb + (size_t)L * 4, (void**)&meta));
    rt.d_scnt = reinterpret_cast<unsigned long long*>(meta);
    rt.d_rcnt = reinterpret_cast<unsigned long long*>(meta + cb);
    rt.d_ovf = reinterpret_cast<uint32_t*>(meta + 2 * cb);
    GTS_CUDA(cudaMemsetAsync(meta, 0, 2 * cb + (size_t)L * 4, c->stream));
    return GTS_OK;
}

}  // namespace gts
