// Page sweeps: resident pages, or pages streamed from pinned host memory
// through a device ring.
//
// Paper (Fig 2/3): topology pages are copied to the GPU
// asynchronously on several streams while kernels process earlier pages;
// copies do not overlap each other but overlap kernel execution; up to
// 32 streams.  B200 design: one copy stream + the compute stream, a
// ring of K slots of B pages each, two events per slot (ready: copy done;
// free: kernel done).  The copy of batch b+K waits only for the kernel of
// batch b, so copies run back to back on the link while kernels trail them.
// Consecutive page ids within a batch are copied by one cudaMemcpyAsync.
#pragma once

#include <algorithm>
#include <vector>

#include "runtime.h"

namespace gts {

constexpr int kBufRing = 60;

struct SweepStats {
    uint64_t h2d_bytes = 0;
    uint64_t launches = 0;
    uint64_t cache_hits = 0;
    uint64_t cache_misses = 0;
};

int ensure_ring(Context* c, const Graph* g, uint32_t slots, uint32_t batch_pages, uint8_t** ring);

// launch(const PageSet& ps, int grid_cap): enqueue the kernel(s) for ps on c->stream.
// Resident: one launch over d_list (nullptr = all local pages in local order)
// with the device-side count d_count (or `count`).  Streamed: h_list holds the
// same page ids on the host (ascending), d_list their device copy.
template <class F>
int sweep_pages(Context* c, const Graph* g, const gts_run_config& rc, bool streamed, const std::vector<uint32_t>* h_list,
                const uint32_t* d_list, uint32_t count, const uint32_t* d_count, F&& launch, SweepStats* ss) {
    const DevGraph& d = c->dg;
    if (!streamed) {
        PageSet ps;
        ps.base = d.pages;
        ps.list = d_list;
        ps.loc = d.loc;
        ps.d_count = d_count;
        ps.count = count;
        ps.page_bytes = g->page_bytes;
        ps.mode = d.all_local ? kAddrByPid : kAddrByLoc;
        ps.entry_encoding = g->entry_encoding;
        ps.rvt_start = d.rvt_start;
        GTS_TRY(launch(ps, 1 << 30));
        ss->launches++;
        return GTS_OK;
    }
    const uint32_t K = rc.ring_slots, B = rc.batch_pages;
    uint8_t* ring;
    GTS_TRY(ensure_ring(c, g, K, B, &ring));
    const size_t pb = g->page_bytes;
    const bool timing = rc.flags & GTS_RUN_TIMING;
    const std::vector<uint32_t>& L = *h_list;
    const uint32_t total = (uint32_t)L.size();
    for (uint32_t b0 = 0, bi = 0; b0 < total; b0 += B, ++bi) {
        const uint32_t slot = bi % K, nb = std::min(B, total - b0);
        uint8_t* dst = ring + (size_t)slot * B * pb;
        GTS_CUDA(cudaStreamWaitEvent(c->copy_stream, c->ring_free[slot], 0));
        std::pair<cudaEvent_t, cudaEvent_t> ev;
        if (timing) {
            ev = c->t_h2d.next();
            cudaEventRecord(ev.first, c->copy_stream);
        }
        uint32_t i = 0;
        while (i < nb) {             // runs of pages adjacent in host memory: one copy each
            const uint8_t* h0 = host_page(g, L[b0 + i]);
            if (!h0) return fail(GTS_EINVAL, "graph does not hold page %u", L[b0 + i]);
            uint32_t j = i + 1;
            while (j < nb && host_page(g, L[b0 + j]) == h0 + (size_t)(j - i) * pb) ++j;
            GTS_CUDA(cudaMemcpyAsync(dst + (size_t)i * pb, h0, (size_t)(j - i) * pb, cudaMemcpyHostToDevice,
                                     c->copy_stream));
            i = j;
        }
        if (timing) cudaEventRecord(ev.second, c->copy_stream);
        GTS_CUDA(cudaEventRecord(c->ring_ready[slot], c->copy_stream));
        GTS_CUDA(cudaStreamWaitEvent(c->stream, c->ring_ready[slot], 0));
        PageSet ps;
        ps.base = dst;
        ps.list = d_list + b0;
        ps.loc = nullptr;
        ps.d_count = nullptr;
        ps.count = nb;
        ps.page_bytes = g->page_bytes;
        ps.mode = kAddrByPos;
        ps.entry_encoding = g->entry_encoding;
        ps.rvt_start = d.rvt_start;
        GTS_TRY(launch(ps, (int)nb));
        GTS_CUDA(cudaEventRecord(c->ring_free[slot], c->stream));
        ss->h2d_bytes += (uint64_t)nb * pb;
        ss->launches++;
    }
    return GTS_OK;
}

constexpr int kBufCacheList = 61;

// Streamed sweep through the LRU page cache: pages of L already cached are
// processed in place (no copy); missing pages are copied into free or least
// recently used slots (never one used in this sweep) in batches of B, each
// batch's kernel waiting for its copy; pages that find no slot take the ring
// path of sweep_pages.
template <class F>
int sweep_pages_cached(Context* c, const Graph* g, const gts_run_config& rc, const std::vector<uint32_t>& L,
                       const uint32_t* d_L, F&& launch, SweepStats* ss) {
    PageCache& pc = c->cache;
    const size_t pb = g->page_bytes;
    const uint32_t want = (uint32_t)std::min<uint64_t>(((uint64_t)rc.cache_mib << 20) / pb, g->num_pages);
    if (pc.uid != g->uid || pc.cap != want || pc.page_bytes != g->page_bytes) {
        free_cache(pc);
        if (want == 0) return sweep_pages(c, g, rc, true, &L, d_L, (uint32_t)L.size(), nullptr, launch, ss);
        cudaError_t e = cudaMalloc(&pc.buf, (size_t)want * pb);
        if (e != cudaSuccess) {
            cudaGetLastError();
            return fail(GTS_ENOMEM, "page cache: cudaMalloc(%zu) failed", (size_t)want * pb);
        }
        GTS_CUDA(cudaMalloc(&pc.d_loc, g->num_pages * 4));
        pc.uid = g->uid;
        pc.cap = want;
        pc.page_bytes = g->page_bytes;
        pc.loc.assign(g->num_pages, UINT32_MAX);
        pc.pid_of.assign(want, UINT32_MAX);
        pc.stamp.assign(want, 0);
        pc.tick = 0;
    }
    const uint64_t tick = ++pc.tick;
    std::vector<uint32_t> hits, miss;
    for (uint32_t p : L) {
        const uint32_t sl = pc.loc[p];
        if (sl != UINT32_MAX) {
            hits.push_back(p);
            pc.stamp[sl] = tick;
        } else {
            miss.push_back(p);
        }
    }
    // victims: free slots first, then least recently used slots not touched in this sweep
    std::vector<uint32_t> cand;
    for (uint32_t sl = 0; sl < pc.cap; ++sl)
        if (pc.stamp[sl] < tick || pc.pid_of[sl] == UINT32_MAX) cand.push_back(sl);
    const size_t ncached = std::min(cand.size(), miss.size());
    if (ncached < cand.size())
        std::nth_element(cand.begin(), cand.begin() + ncached, cand.end(), [&](uint32_t a, uint32_t b) {
            const bool fa = pc.pid_of[a] == UINT32_MAX, fb = pc.pid_of[b] == UINT32_MAX;
            return fa != fb ? fa : pc.stamp[a] < pc.stamp[b];
        });
    for (size_t k = 0; k < ncached; ++k) {
        const uint32_t sl = cand[k], p = miss[k];
        if (pc.pid_of[sl] != UINT32_MAX) pc.loc[pc.pid_of[sl]] = UINT32_MAX;
        pc.pid_of[sl] = p;
        pc.loc[p] = sl;
        pc.stamp[sl] = tick;
    }
    ss->cache_hits += hits.size();
    ss->cache_misses += miss.size();
    // device list = [hits | cached misses]; the loc map goes up with it (the host synchronised
    // after the previous level, so no kernel still reads the slots or the map)
    std::vector<uint32_t> order(hits);
    order.insert(order.end(), miss.begin(), miss.begin() + ncached);
    uint32_t* d_list = nullptr;
    GTS_TRY(c->buf(kBufCacheList, std::max<size_t>(order.size(), 1) * 4, (void**)&d_list));
    if (!order.empty())
        GTS_CUDA(cudaMemcpyAsync(d_list, order.data(), order.size() * 4, cudaMemcpyHostToDevice, c->stream));
    GTS_CUDA(cudaMemcpyAsync(pc.d_loc, pc.loc.data(), g->num_pages * 4, cudaMemcpyHostToDevice, c->stream));
    GTS_CUDA(cudaStreamSynchronize(c->stream));   // host vectors are reused below
    auto cached_set = [&](uint32_t first, uint32_t cnt) {
        PageSet ps;
        ps.base = pc.buf;
        ps.list = d_list + first;
        ps.loc = pc.d_loc;
        ps.d_count = nullptr;
        ps.count = cnt;
        ps.page_bytes = g->page_bytes;
        ps.mode = kAddrByLoc;
        ps.entry_encoding = g->entry_encoding;
        ps.rvt_start = c->dg.rvt_start;
        return ps;
    };
    if (!hits.empty()) {                          // overlaps the miss copies below
        GTS_TRY(launch(cached_set(0, (uint32_t)hits.size()), (int)hits.size()));
        ss->launches++;
    }
    GTS_TRY(ensure_ring(c, g, rc.ring_slots, rc.batch_pages, nullptr));
    const uint32_t B = rc.batch_pages;
    for (size_t b0 = 0, bi = 0; b0 < ncached; b0 += B, ++bi) {
        const uint32_t nb = (uint32_t)std::min<size_t>(B, ncached - b0);
        const uint32_t ev = bi % rc.ring_slots;
        for (uint32_t k = 0; k < nb; ++k) {
            const uint32_t p = miss[b0 + k];
            const uint8_t* hp = host_page(g, p);
            if (!hp) return fail(GTS_EINVAL, "graph does not hold page %u", p);
            GTS_CUDA(cudaMemcpyAsync(pc.buf + (size_t)pc.loc[p] * pb, hp, pb, cudaMemcpyHostToDevice, c->copy_stream));
        }
        GTS_CUDA(cudaEventRecord(c->ring_ready[ev], c->copy_stream));
        GTS_CUDA(cudaStreamWaitEvent(c->stream, c->ring_ready[ev], 0));
        GTS_TRY(launch(cached_set((uint32_t)(hits.size() + b0), nb), (int)nb));
        ss->h2d_bytes += (uint64_t)nb * pb;
        ss->launches++;
    }
    if (ncached < miss.size()) {                  // no slot left: stream the rest through the ring
        std::vector<uint32_t> rest(miss.begin() + ncached, miss.end());
        uint32_t* d_rest = nullptr;
        GTS_TRY(c->buf(kBufCacheList + 1, rest.size() * 4, (void**)&d_rest));
        GTS_CUDA(cudaMemcpyAsync(d_rest, rest.data(), rest.size() * 4, cudaMemcpyHostToDevice, c->stream));
        GTS_CUDA(cudaStreamSynchronize(c->stream));
        GTS_TRY(sweep_pages(c, g, rc, true, &rest, d_rest, (uint32_t)rest.size(), nullptr, launch, ss));
    }
    return GTS_OK;
}

}  // namespace gts
