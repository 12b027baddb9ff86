// Context, device graph residency, page partitioning (Strategy-P / -S), NCCL.
//
// Paper: Alg 1 lines 2-3 create streams and device buffers per GPU;
// Strategy-P copies a different set of pages to each GPU with h(j) = j mod N
// (P:346-354), Strategy-S gives each GPU a different WA chunk.
// B200: one process per GPU (torchrun), one context per process; NCCL comm
// from a unique id broadcast by the caller's process group.
#include <cuda_runtime.h>
#include <nccl.h>

#include <algorithm>
#include <cstring>
#include <new>

#include "memops.cuh"
#include "runtime.h"

namespace gts {

std::pair<cudaEvent_t, cudaEvent_t> Timer::next() {
    if (used == pairs.size()) {
        cudaEvent_t a, b;
        cudaEventCreate(&a);
        cudaEventCreate(&b);
        pairs.emplace_back(a, b);
    }
    return pairs[used++];
}

double Timer::sum_s() {
    double s = 0;
    for (size_t i = 0; i < used; ++i) {
        float ms = 0;
        if (cudaEventElapsedTime(&ms, pairs[i].first, pairs[i].second) == cudaSuccess) s += ms * 1e-3;
    }
    used = 0;
    return s;
}

int Context::buf(int slot, size_t bytes, void** out) {
    if ((size_t)slot >= scratch.size()) scratch.resize(slot + 1, {nullptr, 0});
    auto& b = scratch[slot];
    if (b.second < bytes) {
        if (b.first) cudaFree(b.first);
        b.first = nullptr;
        b.second = 0;
        size_t sz = bytes < 256 ? 256 : bytes;
        cudaError_t e = cudaMalloc(&b.first, sz);
        if (e != cudaSuccess) {
            cudaGetLastError();
            return fail(GTS_ENOMEM, "cudaMalloc(%zu) for scratch slot %d: %s", sz, slot, cudaGetErrorString(e));
        }
        b.second = sz;
    }
    *out = b.first;
    return GTS_OK;
}

// Pin the graph's host pages (and, for ordered graphs, the VID maps) once, so
// uploads and streamed sweeps run at the link rate.  Failure is not an error:
// pageable sources are still correct, only slower.
int pinned_register(Graph* g) {
    if (g->host_registered || g->pages_alloc == 0) return GTS_OK;
    cudaError_t e = cudaHostRegister(g->pages, (g->pages_alloc + 4095) & ~(size_t)4095, cudaHostRegisterPortable);
    if (e != cudaSuccess) {
        cudaGetLastError();
        return GTS_OK;
    }
    g->host_registered = true;
    if (g->ordered) {
        if (cudaHostRegister(g->new_of_old.data(), g->n * 4, cudaHostRegisterPortable) == cudaSuccess &&
            cudaHostRegister(g->old_of_new.data(), g->n * 4, cudaHostRegisterPortable) == cudaSuccess)
            g->maps_registered = true;
        else
            cudaGetLastError();
    }
    return GTS_OK;
}

void free_cache(PageCache& pc) {
    cudaFree(pc.buf);
    cudaFree(pc.d_loc);
    pc = PageCache();
}

static void free_devgraph(DevGraph& d) {
    cudaFree(d.pages);
    cudaFree(d.rvt_start);
    cudaFree(d.nslots);
    cudaFree(d.loc);
    cudaFree(d.local_list);
    cudaFree(d.hot_keys);
    cudaFree(d.new_of_old);
    cudaFree(d.old_of_new);
    d = DevGraph();
}

int ensure_graph(Context* c, const Graph* gc, uint32_t strategy, bool need_resident, double* upload_s) {
    Graph* g = const_cast<Graph*>(gc);
    double t0 = now_s();
    uint32_t strat_key = c->world > 1 ? strategy : 0;
    if (c->dg.uid != g->uid || c->dg.strategy != strat_key || c->dg.world != c->world) {
        if (c->dg.uid) {                              // park the current graph, bring back g if parked
            c->parked.push_back(std::move(c->dg));
            c->dg = DevGraph();
        }
        for (size_t i = 0; i < c->parked.size(); ++i)
            if (c->parked[i].uid == g->uid && c->parked[i].strategy == strat_key && c->parked[i].world == c->world) {
                c->dg = std::move(c->parked[i]);
                c->parked.erase(c->parked.begin() + i);
                break;
            }
    }
    if (c->dg.uid != g->uid) {
        DevGraph& d = c->dg;
        // d.uid is set only after every allocation and upload below succeeded: a failed
        // setup leaves uid = 0, and its partial allocations are freed on the next call
        free_devgraph(d);
        std::vector<uint64_t> vrange;
        partition(g, strategy, c->world, d.h_owner, vrange);
        d.vlo = vrange[c->rank];
        d.vhi = vrange[c->rank + 1];
        d.h_vrange = vrange;
        const uint64_t P = g->num_pages;
        std::vector<uint32_t> loc(P, UINT32_MAX);
        d.h_local_list.clear();
        const bool every_page = strategy == GTS_STRATEGY_S_BCAST;   // each rank streams all pages
        for (uint64_t j = 0; j < P; ++j)
            if (every_page || d.h_owner[j] == c->rank) {
                loc[j] = (uint32_t)d.h_local_list.size();
                d.h_local_list.push_back((uint32_t)j);
            }
        d.n_local = (uint32_t)d.h_local_list.size();
        d.all_local = d.n_local == P;
        GTS_CUDA(cudaMalloc(&d.rvt_start, std::max<size_t>(P, 1) * 4));
        GTS_CUDA(cudaMalloc(&d.nslots, std::max<size_t>(P, 1) * 4));
        GTS_CUDA(cudaMalloc(&d.loc, std::max<size_t>(P, 1) * 4));
        GTS_CUDA(cudaMalloc(&d.local_list, std::max<size_t>(d.n_local, 1) * 4));
        GTS_CUDA(cudaMalloc(&d.hot_keys, kHotSlots * 4));
        GTS_CUDA(cudaMemcpyAsync(d.rvt_start, g->start_vid.data(), P * 4, cudaMemcpyHostToDevice, c->stream));
        GTS_CUDA(cudaMemcpyAsync(d.nslots, g->nslots.data(), P * 4, cudaMemcpyHostToDevice, c->stream));
        GTS_CUDA(cudaMemcpyAsync(d.loc, loc.data(), P * 4, cudaMemcpyHostToDevice, c->stream));
        if (d.n_local)
            GTS_CUDA(cudaMemcpyAsync(d.local_list, d.h_local_list.data(), d.n_local * 4ull, cudaMemcpyHostToDevice,
                                     c->stream));
        GTS_CUDA(cudaMemcpyAsync(d.hot_keys, g->hot_keys.data(), kHotSlots * 4, cudaMemcpyHostToDevice, c->stream));
        if (g->ordered) {
            GTS_TRY(pinned_register(g));
            // old_of_new is uploaded on first use (WCC label renaming in deliver)
            GTS_CUDA(cudaMalloc(&d.new_of_old, g->n * 4));
            GTS_CUDA(cudaMemcpyAsync(d.new_of_old, g->new_of_old.data(), g->n * 4, cudaMemcpyHostToDevice, c->stream));
        }
        GTS_CUDA(cudaStreamSynchronize(c->stream));   // host vectors above are temporaries
        d.uid = g->uid;
        d.strategy = strat_key;
        d.world = c->world;
    }
    DevGraph& d = c->dg;
    if (need_resident && !d.resident) {
        GTS_TRY(pinned_register(g));
        const size_t pb = g->page_bytes;
        d.pages_bytes = (size_t)d.n_local * pb;
        cudaError_t e = cudaMalloc(&d.pages, std::max<size_t>(d.pages_bytes, 256));
        while (e != cudaSuccess && !c->parked.empty()) {   // make room: drop the oldest parked graph
            cudaGetLastError();
            free_devgraph(c->parked.front());
            c->parked.erase(c->parked.begin());
            e = cudaMalloc(&d.pages, std::max<size_t>(d.pages_bytes, 256));
        }
        if (e != cudaSuccess) {
            cudaGetLastError();
            return fail(GTS_ENOMEM, "resident pages: cudaMalloc(%zu) failed: %s", d.pages_bytes,
                        cudaGetErrorString(e));
        }
        // copy runs of pages adjacent in host memory in one cudaMemcpyAsync each
        uint32_t i = 0;
        while (i < d.n_local) {
            const uint8_t* h0 = host_page(g, d.h_local_list[i]);
            if (!h0) return fail(GTS_EINVAL, "graph does not hold page %u of this rank", d.h_local_list[i]);
            uint32_t j = i + 1;
            while (j < d.n_local && host_page(g, d.h_local_list[j]) == h0 + (size_t)(j - i) * pb) ++j;
            GTS_CUDA(cudaMemcpyAsync(d.pages + (size_t)i * pb, h0, (size_t)(j - i) * pb, cudaMemcpyHostToDevice,
                                     c->stream));
            i = j;
        }
        GTS_CUDA(cudaStreamSynchronize(c->stream));
        d.resident = true;
        if (upload_s) *upload_s = now_s() - t0;
    }
    return GTS_OK;
}

int ensure_ring(Context* c, const Graph* g, uint32_t slots, uint32_t batch_pages, uint8_t** ring) {
    GTS_TRY(pinned_register(const_cast<Graph*>(g)));
    if (!c->ring_events) {
        for (int i = 0; i < 64; ++i) {
            GTS_CUDA(cudaEventCreateWithFlags(&c->ring_ready[i], cudaEventDisableTiming));
            GTS_CUDA(cudaEventCreateWithFlags(&c->ring_free[i], cudaEventDisableTiming));
        }
        c->ring_events = true;
    }
    if (!ring) return GTS_OK;    // events only
    return c->buf(60 /* kBufRing */, (size_t)slots * batch_pages * g->page_bytes, (void**)ring);
}

bool choose_streamed(Context* c, const Graph* g, const gts_run_config& rc, uint64_t attr_bytes) {
    if (rc.residency == GTS_STREAMED) return true;
    if (rc.residency == GTS_RESIDENT) return false;
    if (c->dg.uid == g->uid && c->dg.resident) return false;
    // a parked resident copy comes back without an upload (ensure_graph).  (cudaMemGetInfo
    // below measured 1-27 ms per call on B200: asked on every switch between two graphs, it
    // was the per-call outliers of SSSP and WCC in the bench step, tools/call_jitter.py)
    uint32_t strat_key = c->world > 1 ? rc.strategy : 0;
    for (const DevGraph& p : c->parked)
        if (p.uid == g->uid && p.resident && p.strategy == strat_key && p.world == c->world) return false;
    size_t free_b = 0, total_b = 0;
    if (cudaMemGetInfo(&free_b, &total_b) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    uint64_t P = g->num_pages, local = c->world > 1 ? (P + c->world - 1) / c->world : P;
    uint64_t need = local * g->page_bytes + attr_bytes + (1ull << 30);
    return need > free_b;
}

int validate_common(gts_context* ctx, const gts_graph* g, const gts_run_config* cfg, gts_run_config* out) {
    if (!ctx || !g) return fail(GTS_EINVAL, "NULL context or graph");
    gts_run_config d;
    std::memset(&d, 0, sizeof(d));
    d.struct_size = sizeof(d);
    d.strategy = GTS_STRATEGY_P;
    d.residency = GTS_RESIDENCY_AUTO;
    if (cfg) {   // struct_size 32 = the 1.0 layout (the 1.1 fields take their defaults); 0 = current
        const uint32_t sz = cfg->struct_size ? cfg->struct_size : (uint32_t)sizeof(gts_run_config);
        if (sz < 32) return fail(GTS_EINVAL, "gts_run_config.struct_size too small");
        std::memcpy(&d, cfg, std::min<size_t>(sz, sizeof(d)));
        d.struct_size = sizeof(d);
    }
    if (d.strategy > GTS_STRATEGY_S_BCAST) return fail(GTS_EINVAL, "unknown strategy %u", d.strategy);
    if (d.residency > GTS_STREAMED) return fail(GTS_EINVAL, "unknown residency %u", d.residency);
    if (d.out_location > GTS_OUT_DEVICE) return fail(GTS_EINVAL, "unknown out_location %u", d.out_location);
    if (d.virtual_ranks > 8) return fail(GTS_EINVAL, "virtual_ranks must be <= 8");
    if (d.virtual_ranks > 1 && ctx->world > 1) return fail(GTS_EINVAL, "virtual_ranks needs a world-1 context");
    const bool multi = ctx->world > 1 || d.virtual_ranks > 1;
    if (multi && (d.flags & GTS_MICRO_MASK))
        return fail(GTS_EUNSUPPORTED, "GTS_MICRO_* techniques run on one rank");
    if (multi && d.cache_mib) return fail(GTS_EUNSUPPORTED, "the page cache (cache_mib) runs on one rank");
    // an owner-filtered graph holds one rank's pages: only that rank of that job can use it
    if (g->owner_rank >= 0 && g->owner_world > 1 && g->owner_strategy != GTS_STRATEGY_S_BCAST) {
        if (ctx->world != (int)g->owner_world || ctx->rank != g->owner_rank ||
            (ctx->world > 1 && d.strategy != g->owner_strategy))
            return fail(GTS_EINVAL, "graph holds the pages of rank %d/%u (strategy %u); context is rank %d/%d "
                        "(strategy %u)", g->owner_rank, g->owner_world, g->owner_strategy, ctx->rank, ctx->world,
                        d.strategy);
    }
    if (d.ring_slots == 0) d.ring_slots = 4;
    if (d.batch_pages == 0) {   // >= 64 MiB per batch: enough pages in flight to keep the link busy
        const uint32_t pb = g->page_bytes;
        d.batch_pages = pb >= (64u << 20) ? 1u : std::max(8u, (64u << 20) / pb);
        d.batch_pages = std::min<uint32_t>(d.batch_pages, 256);
    }
    if (d.ring_slots > 32) return fail(GTS_EINVAL, "ring_slots must be <= 32");
    *out = d;
    cudaError_t e = cudaSetDevice(ctx->device);
    if (e != cudaSuccess) return fail(GTS_ECUDA, "cudaSetDevice(%d): %s", ctx->device, cudaGetErrorString(e));
    return GTS_OK;
}

// Result D2H (Alg 1 line 28, "copy WA back").  Device outputs: one D2D copy.
// Pinned host outputs: one DMA.  Pageable host outputs: DMA into two pinned
// staging chunks, each drained by a parallel host memcpy while the next chunk
// is in flight (a plain cudaMemcpy to pageable memory runs at a few GB/s).
int copy_out(Context* c, const void* dsrc, void* dst, size_t bytes, uint32_t out_location) {
    if (bytes == 0) return GTS_OK;
    if (out_location == GTS_OUT_DEVICE) {
        GTS_CUDA(cudaMemcpyAsync(dst, dsrc, bytes, cudaMemcpyDeviceToDevice, c->stream));
        GTS_CUDA(cudaStreamSynchronize(c->stream));
        return GTS_OK;
    }
    cudaPointerAttributes pa;
    bool pinned = cudaPointerGetAttributes(&pa, dst) == cudaSuccess && pa.type == cudaMemoryTypeHost;
    cudaGetLastError();
    if (pinned || bytes <= (1u << 20)) {
        GTS_CUDA(cudaMemcpyAsync(dst, dsrc, bytes, cudaMemcpyDeviceToHost, c->stream));
        GTS_CUDA(cudaStreamSynchronize(c->stream));
        return GTS_OK;
    }
    const size_t chunk = 32u << 20;
    if (!c->h_stage) GTS_CUDA(cudaMallocHost(&c->h_stage, 2 * chunk));
    if (!c->stage_ev[0]) {
        GTS_CUDA(cudaEventCreateWithFlags(&c->stage_ev[0], cudaEventDisableTiming));
        GTS_CUDA(cudaEventCreateWithFlags(&c->stage_ev[1], cudaEventDisableTiming));
    }
    const uint8_t* src = static_cast<const uint8_t*>(dsrc);
    uint8_t* out = static_cast<uint8_t*>(dst);
    const size_t nchunks = (bytes + chunk - 1) / chunk;
    auto issue = [&](size_t k) -> int {
        const size_t off = k * chunk, len = std::min(chunk, bytes - off);
        GTS_CUDA(cudaMemcpyAsync(c->h_stage + (k & 1) * chunk, src + off, len, cudaMemcpyDeviceToHost, c->stream));
        GTS_CUDA(cudaEventRecord(c->stage_ev[k & 1], c->stream));
        return GTS_OK;
    };
    GTS_TRY(issue(0));
    for (size_t k = 0; k < nchunks; ++k) {
        if (k + 1 < nchunks) GTS_TRY(issue(k + 1));
        GTS_CUDA(cudaEventSynchronize(c->stage_ev[k & 1]));
        const size_t off = k * chunk, len = std::min(chunk, bytes - off);
        const uint8_t* st = c->h_stage + (k & 1) * chunk;
        const int T = 8;
        #pragma omp parallel for num_threads(T) schedule(static)
        for (int t = 0; t < T; ++t) {
            const size_t a = len * t / T, b = len * (t + 1) / T;
            std::memcpy(out + off + a, st + a, b - a);
        }
    }
    return GTS_OK;
}

__global__ void gather_kernel(uint32_t* out, const uint32_t* __restrict__ vals, const uint32_t* __restrict__ idx,
                              uint64_t n) {
    gather_x4(out, idx, n, [&](uint32_t i) { return __ldg(vals + i); });
}

// min caller VID per component.  Each thread folds runs of equal labels in a
// register before touching memory (a giant component shares one label, and a
// read or atomic per vertex on that one address serialises on one L2 slice).
__device__ __forceinline__ void label_min_flush(uint32_t* minorig, uint32_t l, uint32_t o) {
    if (o < __ldcg(minorig + l)) atomicMin(minorig + l, o);
}

__global__ void label_min_kernel(uint32_t* minorig, const uint32_t* __restrict__ label,
                                 const uint32_t* __restrict__ old_of_new, uint64_t n) {
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    const uint64_t t = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    uint32_t cl = 0xFFFFFFFFu, cm = 0xFFFFFFFFu;
    auto fold = [&](uint32_t l, uint32_t o) {
        if (l == cl) {
            cm = min(cm, o);
        } else {
            if (cl != 0xFFFFFFFFu) label_min_flush(minorig, cl, cm);
            cl = l;
            cm = o;
        }
    };
    // four consecutive vertices per step with 16-byte loads; the tail (or
    // everything, if an array is not 16-byte aligned) element by element
    const bool al = ((((uintptr_t)label) | ((uintptr_t)old_of_new)) & 15u) == 0;
    const uint64_t n4 = al ? n >> 2 : 0;
    for (uint64_t q = t; q < n4; q += stride) {
        const uint4 l = __ldcs(reinterpret_cast<const uint4*>(label) + q);
        const uint4 o = __ldcs(reinterpret_cast<const uint4*>(old_of_new) + q);
        fold(l.x, o.x);
        fold(l.y, o.y);
        fold(l.z, o.z);
        fold(l.w, o.w);
    }
    for (uint64_t i = 4 * n4 + t; i < n; i += stride) fold(label[i], old_of_new[i]);
    if (cl != 0xFFFFFFFFu) label_min_flush(minorig, cl, cm);
}

// label_map + gather in one pass: out[v] = minorig[label[new_of_old[v]]] (caller order)
__global__ void label_gather_kernel(uint32_t* out, const uint32_t* __restrict__ label,
                                    const uint32_t* __restrict__ minorig, const uint32_t* __restrict__ idx,
                                    uint64_t n) {
    gather_x4(out, idx, n, [&](uint32_t i) { return __ldg(minorig + __ldg(label + i)); });
}

int ensure_old_of_new(Context* c, const Graph* g, const uint32_t** out) {
    if (!c->dg.old_of_new) {
        GTS_CUDA(cudaMalloc(&c->dg.old_of_new, g->n * 4));
        GTS_CUDA(cudaMemcpyAsync(c->dg.old_of_new, g->old_of_new.data(), g->n * 4, cudaMemcpyHostToDevice, c->stream));
    }
    *out = c->dg.old_of_new;
    return GTS_OK;
}

int deliver(Context* c, const Graph* g, const uint32_t* vals, void* out, uint32_t out_location, bool labels) {
    const uint64_t n = g->n;
    if (!g->ordered) return copy_out(c, vals, out, n * 4, out_location);
    const int eg = c->num_sms * 4;
    uint32_t* minorig = nullptr;
    if (labels) {             // internal min-ID label -> min caller VID of the component
        const uint32_t* onew;
        GTS_TRY(ensure_old_of_new(c, g, &onew));
        GTS_TRY(c->buf(70, n * 4, (void**)&minorig));
        GTS_CUDA(cudaMemsetAsync(minorig, 0xFF, n * 4, c->stream));
        label_min_kernel<<<eg, 256, 0, c->stream>>>(minorig, vals, c->dg.old_of_new, n);
    }
    uint32_t* dst;
    if (out_location == GTS_OUT_DEVICE) dst = static_cast<uint32_t*>(out);
    else GTS_TRY(c->buf(72, n * 4, (void**)&dst));
    if (labels) label_gather_kernel<<<2 * eg, 256, 0, c->stream>>>(dst, vals, minorig, c->dg.new_of_old, n);
    else gather_kernel<<<2 * eg, 256, 0, c->stream>>>(dst, vals, c->dg.new_of_old, n);
    GTS_CUDA(cudaGetLastError());
    if (out_location == GTS_OUT_DEVICE) {
        GTS_CUDA(cudaStreamSynchronize(c->stream));
        return GTS_OK;
    }
    return copy_out(c, dst, out, n * 4, out_location);
}

int persist_window(Context* c, cudaStream_t s, void* p, size_t bytes) {
    cudaStreamAttrValue at;
    std::memset(&at, 0, sizeof(at));
    if (p && bytes) {
        const size_t want = std::min(bytes, c->persist_max);
        if (want == 0) return GTS_OK;
        if (c->persist_limit != c->persist_max) {   // device-wide set-aside: the maximum, set once
            GTS_CUDA(cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, c->persist_max));
            c->persist_limit = c->persist_max;
        }
        at.accessPolicyWindow.base_ptr = p;
        at.accessPolicyWindow.num_bytes = std::min(want, c->window_max);
        at.accessPolicyWindow.hitRatio = 1.0f;
        at.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
        at.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
    }
    GTS_CUDA(cudaStreamSetAttribute(s, cudaStreamAttributeAccessPolicyWindow, &at));
    return GTS_OK;
}

int sms_grid(Context* c, const void* kernel, int threads, size_t smem, int* grid) {
    int per_sm = 0;
    GTS_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kernel, threads, smem));
    if (per_sm < 1) per_sm = 1;
    *grid = per_sm * c->num_sms;
    return GTS_OK;
}

}  // namespace gts

using namespace gts;

extern "C" int gts_get_unique_id(uint8_t out[128]) {
    clear_error();
    if (!out) return fail(GTS_EINVAL, "NULL out");
    ncclUniqueId id;
    GTS_NCCL(ncclGetUniqueId(&id));
    static_assert(sizeof(id) == 128, "ncclUniqueId is 128 bytes");
    std::memcpy(out, &id, 128);
    return GTS_OK;
}

extern "C" int gts_context_create(int device, int rank, int world_size, const uint8_t* unique_id,
                                  gts_context** out) {
    clear_error();
    if (!out) return fail(GTS_EINVAL, "NULL out");
    *out = nullptr;
    if (world_size < 1 || rank < 0 || rank >= world_size) return fail(GTS_EINVAL, "bad rank/world_size");
    if (world_size > 1 && !unique_id) return fail(GTS_EINVAL, "world_size > 1 needs an NCCL unique id");
    int ndev = 0;
    cudaError_t e = cudaGetDeviceCount(&ndev);
    if (e != cudaSuccess || ndev == 0) {
        cudaGetLastError();
        return fail(GTS_ECUDA, "no CUDA device available (%s); libgts has no CPU fallback",
                    cudaGetErrorString(e));
    }
    if (device < 0 || device >= ndev) return fail(GTS_EINVAL, "device %d out of range (%d devices)", device, ndev);
    GTS_CUDA(cudaSetDevice(device));
    gts_context* c = new (std::nothrow) gts_context();
    if (!c) return fail(GTS_ENOMEM, "context alloc");
    c->device = device;
    c->rank = rank;
    c->world = world_size;
    cudaDeviceProp prop;
    GTS_CUDA(cudaGetDeviceProperties(&prop, device));
    c->num_sms = prop.multiProcessorCount;
    c->persist_max = prop.persistingL2CacheMaxSize;
    c->window_max = prop.accessPolicyMaxWindowSize;
    GTS_CUDA(cudaStreamCreateWithFlags(&c->own_stream, cudaStreamNonBlocking));
    GTS_CUDA(cudaStreamCreateWithFlags(&c->copy_stream, cudaStreamNonBlocking));
    c->stream = c->own_stream;
    GTS_CUDA(cudaMallocHost(&c->h_small, 4096));
    if (world_size > 1) {
        ncclUniqueId id;
        std::memcpy(&id, unique_id, sizeof(id));
        ncclResult_t r = ncclCommInitRank(&c->comm, world_size, id, rank);
        if (r != ncclSuccess) {
            delete c;
            return fail(GTS_ENCCL, "ncclCommInitRank: %s", ncclGetErrorString(r));
        }
    }
    *out = c;
    return GTS_OK;
}

extern "C" void gts_context_free(gts_context* c) {
    if (!c) return;
    cudaSetDevice(c->device);
    cudaDeviceSynchronize();
    free_devgraph(c->dg);
    for (auto& d : c->parked) free_devgraph(d);
    free_cache(c->cache);
    for (auto& kv : c->ipc_open) cudaIpcCloseMemHandle(kv.second);
    for (auto& b : c->scratch) cudaFree(b.first);
    for (Timer* t : {&c->t_main, &c->t_finish, &c->t_merge, &c->t_h2d})
        for (auto& p : t->pairs) {
            cudaEventDestroy(p.first);
            cudaEventDestroy(p.second);
        }
    if (c->ring_events)
        for (int i = 0; i < 64; ++i) {
            cudaEventDestroy(c->ring_ready[i]);
            cudaEventDestroy(c->ring_free[i]);
        }
    if (c->persist_limit) cudaCtxResetPersistingL2Cache();
    if (c->comm) ncclCommDestroy(c->comm);
    cudaFreeHost(c->h_small);
    if (c->h_stage) cudaFreeHost(c->h_stage);
    for (cudaEvent_t e : c->stage_ev)
        if (e) cudaEventDestroy(e);
    cudaStreamDestroy(c->own_stream);
    cudaStreamDestroy(c->copy_stream);
    delete c;
}

extern "C" int gts_context_evict(gts_context* c, const gts_graph* g) {
    clear_error();
    if (!c) return fail(GTS_EINVAL, "NULL context");
    cudaSetDevice(c->device);
    cudaStreamSynchronize(c->stream);
    if (!g || c->dg.uid == g->uid) free_devgraph(c->dg);
    if (!g || c->cache.uid == g->uid) free_cache(c->cache);
    for (size_t i = c->parked.size(); i-- > 0;)
        if (!g || c->parked[i].uid == g->uid) {
            free_devgraph(c->parked[i]);
            c->parked.erase(c->parked.begin() + i);
        }
    return GTS_OK;
}

extern "C" int gts_context_set_stream(gts_context* c, void* s) {
    clear_error();
    if (!c) return fail(GTS_EINVAL, "NULL context");
    c->stream = s ? (cudaStream_t)s : c->own_stream;
    return GTS_OK;
}

extern "C" void gts_graph_free(gts_graph* g) {
    if (!g) return;
    if (g->host_registered) cudaHostUnregister(g->pages);
    if (g->maps_registered) {
        cudaHostUnregister(g->new_of_old.data());
        cudaHostUnregister(g->old_of_new.data());
    }
    std::free(g->pages);
    delete g;
}

extern "C" int gts_partition_pages(const gts_graph* g, uint32_t strategy, int world_size, int32_t* owner,
                                   uint64_t* vrange) {
    clear_error();
    if (!g || !owner || world_size < 1) return fail(GTS_EINVAL, "bad argument");
    if (strategy > GTS_STRATEGY_S_BCAST) return fail(GTS_EINVAL, "unknown strategy");
    std::vector<int32_t> o;
    std::vector<uint64_t> vr;
    partition(g, strategy, world_size, o, vr);
    std::memcpy(owner, o.data(), o.size() * 4);
    if (vrange) std::memcpy(vrange, vr.data(), vr.size() * 8);
    return GTS_OK;
}
