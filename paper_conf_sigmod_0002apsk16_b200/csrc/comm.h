// The ranks of one call and the merges between them.
//
// Paper: Strategy-P merges the replicated WA of every GPU after each
// iteration / level; Strategy-S splits WA into per-GPU chunks
// (P:430-440).  B200 design: one process per GPU, NCCL
// over NVLink for the merges.  A call runs the ranks of its job that live in
// this process:
//   * a real rank (world > 1): one local slot, collectives are NCCL calls on
//     the context's communicator;
//   * virtual ranks (gts_run_config.virtual_ranks = V > 1 on a world-1
//     context): all V ranks of a V-GPU job run one after another on this GPU,
//     each with its own page set and its own WA buffers, and the collectives
//     are done in device memory.  Every kernel of the multi-GPU path (the
//     per-rank sweeps, the merge kernels, route packing and apply, the
//     capacity exchange) runs exactly as it does on N GPUs; only the
//     transport differs.
#pragma once

#include <array>
#include <vector>

#include "runtime.h"

namespace gts {

constexpr int kMaxRanks = 8;

enum CType : int { kCF32 = 0, kCF64, kCU32, kCU64 };
enum COp : int { kCSum = 0, kCMin, kCMax };

// Routed updates (Strategy-S, SURVEY 8(e) "S-route"): per local slot a send
// buffer with one region per peer (offset + capacity, in messages) and device
// counters the kernels bump; after route_exchange() the receive buffer holds
// every peer's messages for this rank at roff[p], rcnt[p] of them.
struct Route {
    size_t esize = 0;                                         // bytes per message
    std::vector<uint8_t*> send, recv;                         // [nloc]
    std::vector<std::array<uint64_t, kMaxRanks>> soff, scap;  // [nloc][peer]
    std::vector<std::array<uint64_t, kMaxRanks>> roff, rcap;  // [nloc][peer]
    unsigned long long* d_scnt = nullptr;                     // [nloc][kMaxRanks] appended per peer (device)
    unsigned long long* d_rcnt = nullptr;                     // [nloc][kMaxRanks] received per peer (device)
    uint32_t* d_ovf = nullptr;                                // [nloc] a region was full (device)
    std::vector<std::array<uint64_t, kMaxRanks>> h_rcnt;      // host copy of the received counts
    uint64_t sent_msgs = 0;                                   // messages that crossed ranks (stats)
};

struct Ranks {
    Context* c = nullptr;
    int world = 1;      // ranks of the job (N)
    int r0 = 0;         // first rank simulated here
    int nloc = 1;       // local slots: slot i is rank r0 + i
    bool virt = false;  // virtual ranks (in-memory collectives)
    uint64_t bytes = 0; // bytes this process contributed to merges (stats: nccl_bytes)

    int rank(int i) const { return r0 + i; }
    bool multi() const { return world > 1; }

    // In-place reduction of count elements over all ranks; bufs[i] = slot i's buffer.
    int allreduce(void* const* bufs, size_t count, CType t, COp op);
    // recv[i] = send of rank 0 | rank 1 | ... (bytes each).
    int allgather(const void* const* send, void* const* recv, size_t bytes);
    // Every rank r owns elements [vr[r], vr[r+1]) of an n-element array; afterwards every
    // slot's full array holds every owner's range.  full[i] = slot i's array (absolute index).
    int gather_ranges(void* const* full, const std::vector<uint64_t>& vr, size_t esize);
    // Owner-side sum of per-rank partials: for every owner q, dst[q's slot][v] += sum over all
    // ranks of part[rank][v] for v in [a_q, b_q) (a_q, b_q clipped to [0, limit)).
    // part[i] is an f32 array indexed by absolute ID; dst[i] is slot i's biased f32 WA.
    int reduce_to_owners(float* const* part, float* const* dst_biased, const std::vector<uint64_t>& vr,
                         uint64_t limit);
    // Send counts, then messages, between all ranks; fills rt.h_rcnt / rt.d_rcnt.
    int route_exchange(Route& rt);
    // Max over ranks of each slot's overflow flag (returned on the host).
    int route_overflow(Route& rt, bool* any);
    // Peer memory: out[i][q] = rank q's allocation `base[q's slot]` as seen by slot i (virtual
    // ranks: the same pointer; real ranks: a CUDA IPC mapping of the peer's allocation over
    // NVLink, exchanged through an all-gather of the IPC handles and cached in the context).
    // base[i] must be the start of a cudaMalloc allocation of slot i.
    int peer_map(void* const* base, std::vector<std::array<void*, kMaxRanks>>& out);
    // Every rank has reached this point in stream order (an 8-byte all-reduce).
    int barrier();
};

// The ranks this call runs: virtual (V > 1 on a world-1 context), a real rank, or one.
int make_ranks(Context* c, const gts_run_config& rc, Ranks* R);

// Remote edges per (sender rank, owner) of every rank's pages, the capacities of the
// route regions (destinations < skip_below are excluded: PageRank's dense hot set).
// Cached per (graph, strategy, world, skip_below) in the context.  cap[r][p] for all
// ranks (real ranks all-gather their rows).
int route_capacities(Context* c, const Graph* g, Ranks& R, const gts_run_config& rc, bool streamed,
                     const std::vector<std::vector<uint32_t>>& plist, const uint32_t* const* d_plist,
                     const std::vector<uint64_t>& vr, uint32_t skip_below,
                     std::vector<std::array<uint64_t, kMaxRanks>>& cap);

// Allocate rt's send/recv regions from capacities (message size esize) in scratch slots
// [base, base + 2 * nloc).
int route_setup(Context* c, Ranks& R, const std::vector<std::array<uint64_t, kMaxRanks>>& cap, size_t esize,
                int base, Route& rt);

}  // namespace gts
