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
        while (i < nb) {
            uint32_t j = i + 1;
            while (j < nb && L[b0 + j] == L[b0 + j - 1] + 1) ++j;
            GTS_CUDA(cudaMemcpyAsync(dst + (size_t)i * pb, g->pages + (size_t)L[b0 + i] * pb, (size_t)(j - i) * pb,
                                     cudaMemcpyHostToDevice, c->copy_stream));
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

}  // namespace gts
