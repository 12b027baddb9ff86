// Device side of the routed updates of Strategy-S (SURVEY 8(e) "S-route";
// each GPU owns one chunk of WA).  A kernel of rank r applies
// updates whose destination lies in its own WA range [lo, hi) directly and
// appends every other one as a message to the region of the destination's
// owner; comm.cu moves the regions between ranks and the owner applies them.
#pragma once

#include <cstdint>

#include "comm.h"

namespace gts {

struct RouteOut {
    uint8_t* send;                       // this rank's send buffer
    unsigned long long* cnt;             // [kMaxRanks] messages appended per peer
    uint32_t* ovf;                       // set when a region is full (the message is dropped)
    uint64_t vr[kMaxRanks + 1];          // WA ranges: rank p owns [vr[p], vr[p+1])
    uint64_t off[kMaxRanks];             // region of peer p, in messages
    uint64_t cap[kMaxRanks];
    int nranks;
};

__device__ __forceinline__ int route_owner(const RouteOut& ro, uint32_t v) {
    int p = 0;
    while (p < ro.nranks - 1 && (uint64_t)v >= ro.vr[p + 1]) ++p;
    return p;
}

// Append msg for the owner of dst.  Lanes of a warp bound for the same owner
// share one atomic on its counter (__match_any_sync); a full region drops the
// message and raises the overflow flag (capacities are exact upper bounds, so
// this only guards against a counting bug; the call then fails on every rank).
template <class M>
__device__ __forceinline__ void route_push(const RouteOut& ro, uint32_t dst, const M& msg) {
    const int p = route_owner(ro, dst);
    const uint32_t active = __activemask();
    const uint32_t peers = __match_any_sync(active, p);
    const int lane = threadIdx.x & 31;
    const int leader = __ffs(peers) - 1;
    unsigned long long base = 0;
    if (lane == leader) base = atomicAdd(ro.cnt + p, (unsigned long long)__popc(peers));
    base = __shfl_sync(peers, base, leader);
    const unsigned long long slot = base + __popc(peers & ((1u << lane) - 1u));
    if (slot < ro.cap[p]) reinterpret_cast<M*>(ro.send)[ro.off[p] + slot] = msg;
    else *ro.ovf = 1u;
}

}  // namespace gts
