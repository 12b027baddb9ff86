// Context / device-graph state shared by the CUDA translation units.
#pragma once

#include <cuda_runtime.h>
#include <nccl.h>

#include <chrono>
#include <map>
#include <string>
#include <cstdlib>
#include <utility>
#include <vector>

#include "gts_internal.h"

namespace gts {

#define GTS_CUDA(call)                                                                        \
    do {                                                                                      \
        cudaError_t e_ = (call);                                                              \
        if (e_ != cudaSuccess)                                                                \
            return ::gts::fail(GTS_ECUDA, "%s:%d %s: %s", __FILE__, __LINE__, #call,          \
                               cudaGetErrorString(e_));                                       \
    } while (0)

#define GTS_NCCL(call)                                                                        \
    do {                                                                                      \
        ncclResult_t r_ = (call);                                                             \
        if (r_ != ncclSuccess)                                                                \
            return ::gts::fail(GTS_ENCCL, "%s:%d %s: %s", __FILE__, __LINE__, #call,          \
                               ncclGetErrorString(r_));                                       \
    } while (0)

#define GTS_TRY(call)                   \
    do {                                \
        int rc_ = (call);               \
        if (rc_ != GTS_OK) return rc_;  \
    } while (0)

// How a kernel finds the bytes of its i-th work page.
enum PageAddrMode : uint32_t {
    kAddrByPid = 0,   // data = base + pid * page_bytes          (all pages resident in ID order)
    kAddrByLoc = 1,   // data = base + loc[pid] * page_bytes     (this rank's pages resident, compacted)
    kAddrByPos = 2,   // data = base + i * page_bytes            (streamed batch in a ring slot)
};

struct PageSet {
    const uint8_t* base;
    const uint32_t* list;      // global page ids of the work items; nullptr = identity (pid = i)
    const uint32_t* loc;       // kAddrByLoc: page id -> index within base
    const uint32_t* d_count;   // device-side item count (nullptr: use count)
    uint32_t count;
    uint32_t page_bytes;
    uint32_t mode;
    uint32_t entry_encoding;
    const uint32_t* rvt_start; // START_VID per page (PID16 decode)
    uint32_t hybrid_deg = 8;   // GTS_MICRO_HYBRID: vertex-centric below this many edges per vertex (R24)
    uint32_t split = 1;        // work items per page: an LP's chunk is cut into `split` slices
                               // (small page sets, e.g. a hub's LPs at BFS level 0); SPs use slice 0
};

// Device copy of a graph for one rank.
struct DevGraph {
    uint64_t uid = 0;
    uint32_t strategy = 0;
    int world = 1;
    uint8_t* pages = nullptr;          // this rank's resident pages (compacted in local order)
    size_t pages_bytes = 0;
    uint32_t* rvt_start = nullptr;     // [num_pages] START_VID
    uint32_t* nslots = nullptr;        // [num_pages]
    uint32_t* loc = nullptr;           // [num_pages] local index or UINT32_MAX
    uint32_t* local_list = nullptr;    // [n_local] global page ids owned by this rank
    uint32_t* hot_keys = nullptr;      // [kHotSlots]
    uint32_t* new_of_old = nullptr;    // ordered graphs: caller VID -> internal ID  [n]
    uint32_t* old_of_new = nullptr;    // ordered graphs: internal ID -> caller VID  [n]
    uint32_t n_local = 0;
    bool all_local = true;             // every page is local and loc == identity
    bool resident = false;             // pages uploaded
    std::vector<uint32_t> h_local_list;
    std::vector<int32_t> h_owner;
    uint64_t vlo = 0, vhi = 0;         // Strategy-S WA range of this rank
    // binned PageRank scatter: pairs per bin of this rank's pages, for the geometry pb_key
    std::vector<unsigned long long> pb_count;
    uint64_t pb_key = 0;
    std::vector<uint64_t> h_vrange;    // all ranks' WA ranges (world + 1)
    // Strategy-S route capacities (comm.cu route_capacities), per (skip, world, strategy)
    std::map<uint64_t, std::vector<uint64_t>> route_caps;
};

// LRU cache of topology pages in device memory for streamed BFS-like sweeps
// (cachedPIDMap; Alg 1 lines 8, 16, 29).
struct PageCache {
    uint64_t uid = 0;                  // graph the cache holds pages of
    uint32_t cap = 0;                  // slots
    uint32_t page_bytes = 0;
    uint8_t* buf = nullptr;            // cap * page_bytes
    uint32_t* d_loc = nullptr;         // [num_pages] page -> slot (UINT32_MAX = not cached)
    std::vector<uint32_t> loc;         // host mirror of d_loc
    std::vector<uint32_t> pid_of;      // slot -> page (UINT32_MAX = free)
    std::vector<uint64_t> stamp;       // slot -> tick of last use
    uint64_t tick = 0;
};

struct Timer {               // event pairs around launches; summed after the call synchronises
    std::vector<std::pair<cudaEvent_t, cudaEvent_t>> pairs;
    size_t used = 0;
    std::pair<cudaEvent_t, cudaEvent_t> next();
    double sum_s();          // sums pairs[0..used) and resets used
};

struct Context {
    int device = 0, rank = 0, world = 1;
    int num_sms = 148;
    cudaStream_t own_stream = nullptr, stream = nullptr, copy_stream = nullptr;
    ncclComm_t comm = nullptr;
    DevGraph dg;                   // the graph of the current call
    PageCache cache;               // streamed BFS/SSSP page cache
    std::vector<DevGraph> parked;  // other graphs kept resident (evicted LRU-first under memory pressure)
    std::vector<std::pair<void*, size_t>> scratch;
    void* h_small = nullptr;   // pinned host scratch (4 KiB)
    uint8_t* h_stage = nullptr;          // pinned D2H staging (2 x 32 MiB) for pageable outputs
    cudaEvent_t stage_ev[2] = {nullptr, nullptr};
    Timer t_main, t_finish, t_merge, t_h2d;
    cudaEvent_t ring_ready[64], ring_free[64];
    bool ring_events = false;
    uint64_t launches = 0, main_launches = 0;
    std::map<std::string, void*> ipc_open;   // peer allocations opened by handle bytes (GTS_ROUTE_PEER)
    size_t persist_limit = 0;      // cudaLimitPersistingL2CacheSize set by this context
    size_t persist_max = 0;        // device attributes, queried once
    size_t window_max = 0;

    int buf(int slot, size_t bytes, void** out);   // grow-only scratch device buffer
};

// context.cu
int ensure_graph(Context* c, const Graph* g, uint32_t strategy, bool need_resident, double* upload_s);
int validate_common(gts_context* ctx, const gts_graph* g, const gts_run_config* cfg, gts_run_config* out);
int copy_out(Context* c, const void* dsrc, void* dst, size_t bytes, uint32_t out_location);
// Result of a call (internal IDs for ordered graphs) -> caller's buffer in caller VIDs.
// labels = true: the values are themselves internal VIDs (WCC) and are renamed to
// the minimum caller VID of their component.
int deliver(Context* c, const Graph* g, const uint32_t* vals, void* out, uint32_t out_location, bool labels);
// device copy of old_of_new (internal ID -> caller VID), uploaded on first use
int ensure_old_of_new(Context* c, const Graph* g, const uint32_t** out);
inline uint64_t map_src(const Graph* g, uint64_t src) { return g->ordered ? g->new_of_old[src] : src; }
int sms_grid(Context* c, const void* kernel, int threads, size_t smem, int* grid);
// access-policy window on stream s: [p, p + bytes) persisting in L2 (bytes clipped to the
// device limits); p = nullptr clears the window
int persist_window(Context* c, cudaStream_t s, void* p, size_t bytes);
int pinned_register(Graph* g);
void free_cache(PageCache& pc);
// residency decision (GTS_RESIDENCY_AUTO: resident iff this rank's pages + attributes fit in free HBM)
bool choose_streamed(Context* c, const Graph* g, const gts_run_config& rc, uint64_t attr_bytes);


// persisting-L2 window size of a call (gts_run_config.l2_persist_mib: 0 = 96 MiB, GTS_OFF = none)
inline size_t l2_persist_mib(const gts_run_config& rc) {
    return rc.l2_persist_mib == GTS_OFF ? 0 : rc.l2_persist_mib ? rc.l2_persist_mib : 96;
}

inline double now_s() {
    return std::chrono::duration<double>(std::chrono::steady_clock::now().time_since_epoch()).count();
}

}  // namespace gts

struct gts_context : gts::Context {};
