// Internal declarations shared by the libgts translation units (host + device).
// Nothing here is visible through the C ABI (include/gts.h).
#pragma once

#include <cstdint>
#include <cstddef>
#include <string>
#include <vector>

#include "gts.h"

#ifdef __CUDACC__
#define GTS_HD __host__ __device__ __forceinline__
#else
#define GTS_HD inline
#endif

namespace gts {

// ---- error plumbing (capi.cpp) ------------------------------------------
int fail(int code, const char* fmt, ...);          // sets the thread-local message, returns code
void clear_error();

// ---- page layout constants (include/gts.h "Page layout") ----------------
constexpr uint32_t kSpFooter = 8;    // u32 nslots, u32 kind
constexpr uint32_t kLpFooter = 16;   // u32 total_deg, u32 chunk_idx, u32 nslots, u32 kind
constexpr uint32_t kSlotBytes = 8;   // u32 vid, u32 off
constexpr uint32_t kDefaultPageBytes = 1u << 20;
// Record words (include/gts.h "Page layout"): unweighted u32 sz, u32 adj[sz];
// weighted u32 sz, u32 0, then sz (u32 adj, u32 w) pairs, 8-byte aligned, so an
// edge's neighbour and weight are one 8-byte load.
GTS_HD constexpr uint32_t rec_hdr_words(bool weighted) { return weighted ? 2u : 1u; }
GTS_HD constexpr uint32_t rec_edge_words(bool weighted) { return weighted ? 2u : 1u; }

// ---- hot-destination table (PageRank CTA pre-aggregation, DESIGN.md K-PR) ----
// Bucketed two-choice hash table of VIDs; a key lives in bucket h1 if h1 had a
// free way when it was inserted, else in h2.  No deletion, so a lookup may stop
// at h1 when h1 has an empty way.
constexpr uint32_t kHotBuckets = 2048;
constexpr uint32_t kHotWays = 4;
constexpr uint32_t kHotSlots = kHotBuckets * kHotWays;
constexpr uint32_t kHotMax = 4096;          // load factor 0.5
constexpr uint32_t kHotMinIndeg = 64;
constexpr uint32_t kHotEmpty = 0xFFFFFFFFu;
// Degree-ordered graphs: the hot set is simply internal IDs [0, kHotDense).
constexpr uint32_t kHotDense = 24576;

GTS_HD uint32_t hot_h1(uint32_t v) { return (v * 0x9E3779B1u) >> 21; }
GTS_HD uint32_t hot_h2(uint32_t v) { return ((v ^ (v >> 15)) * 0x85EBCA77u) >> 21; }

// ---- graph ---------------------------------------------------------------
struct Graph {
    uint64_t n = 0, m = 0;
    uint32_t page_bytes = 0;
    uint32_t entry_encoding = 0;
    bool weighted = false;
    uint64_t num_pages = 0, n_sp = 0, n_lp = 0, n_lp_vertices = 0, used_bytes = 0, max_outdeg = 0;
    uint8_t* pages = nullptr;          // host, 4 KiB aligned, num_pages * page_bytes
    size_t pages_alloc = 0;
    std::vector<uint32_t> start_vid;   // RVT START_VID
    std::vector<uint32_t> nslots;      // vertices in the page (1 for LP)
    std::vector<uint32_t> kind;        // GTS_PAGE_SP / GTS_PAGE_LP
    std::vector<int64_t> lp_first, lp_last;
    std::vector<uint32_t> hot_keys;    // kHotSlots entries, kHotEmpty when free
    uint32_t n_hot = 0;
    uint64_t uid = 0;                  // process-unique id (device cache key)
    bool ordered = false;              // GTS_BUILD_DEGREE_ORDER: pages hold internal IDs
    std::vector<uint32_t> new_of_old;  // caller VID -> internal ID (ordered graphs)
    std::vector<uint32_t> old_of_new;  // internal ID -> caller VID
    bool host_registered = false;      // pages cudaHostRegister'ed by a context
    bool maps_registered = false;      // new_of_old / old_of_new registered too
    bool symmetric = false;            // GTS_BUILD_SYMMETRIC: every edge stored in both directions
    // GTS_BUILD_OWNER_FILTER: only the pages rank owner_rank of owner_world processes under
    // owner_strategy are held, compacted in ascending page ID; host_loc[pid] = index in pages
    // (UINT32_MAX: not held).  owner_rank = -1: every page held, host_loc empty (identity).
    int32_t owner_rank = -1;
    uint32_t owner_world = 1, owner_strategy = 0;
    std::vector<uint32_t> host_loc;
    uint64_t n_host_pages = 0;
};

// host address of page pid (nullptr if this graph does not hold it)
inline const uint8_t* host_page(const Graph* g, uint64_t pid) {
    if (g->host_loc.empty()) return g->pages + pid * (uint64_t)g->page_bytes;
    const uint32_t l = g->host_loc[pid];
    return l == UINT32_MAX ? nullptr : g->pages + (uint64_t)l * g->page_bytes;
}

// Page -> rank assignment of a strategy (P:352-354 Strategy-P h(j) = j mod N;
// P:430-434 Strategy-S contiguous WA ranges cut at page boundaries with ~equal
// page counts, never inside an LP run).  vrange[world+1]: rank r owns WA
// [vrange[r], vrange[r+1]).  Needs only the directory (n, num_pages, start_vid,
// kind, lp_first).
void partition(const Graph* g, uint32_t strategy, int world, std::vector<int32_t>& owner,
               std::vector<uint64_t>& vrange);

struct PagePlanEntry {
    uint32_t start_vid;
    uint32_t nslots;
    uint32_t kind;
    int64_t lp_first, lp_last;
};

// builder.cpp
int plan_pages(uint64_t n, const uint64_t* row_ptr, bool weighted, uint32_t page_bytes,
               uint32_t entry_encoding, std::vector<PagePlanEntry>& plan, gts_graph_stats* st);

}  // namespace gts

struct gts_graph : gts::Graph {};
