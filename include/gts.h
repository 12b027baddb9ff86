/*
 * gts.h -- C ABI of the B200-native GTS hot path (libgts.so).
 *
 * GTS = "A Fast and Scalable Graph Processing Method based on Streaming
 * Topology to GPUs", Kim et al., SIGMOD'16.  Citations "P:L" refer to line L of
 * the paper text; "R#" to the readings listed in DESIGN.md.
 *
 * The problem statement the calls follow is Algorithm 1's input:
 * a graph G stored as slotted pages, an algorithm (K_SP / K_LP pair), a start
 * vertex for BFS-like algorithms or an iteration count for PageRank-like ones,
 * N GPUs and a multi-GPU strategy.  The algorithms are fixed (BFS,
 * PageRank, SSSP, WCC); there is no user-kernel plug-in.
 *
 * General rules (all functions):
 *   - return int status: GTS_OK (0) or a negative gts_status; no C++
 *     exception ever crosses the ABI; gts_last_error() gives a thread-local
 *     message for the last failing call on the calling thread.
 *   - one call at a time per context; different contexts on different
 *     devices may run concurrently.
 *   - inputs are borrowed for the duration of the call only; outputs are
 *     caller-allocated.
 *   - every call that computes is synchronous: it returns when the result is
 *     in the caller's output buffer (host, or device if GTS_OUT_DEVICE).
 *   - there is no CPU fallback: calls that compute need a CUDA device and
 *     return GTS_ECUDA when none is usable.
 *
 * Page layout (the slotted page of P:64-66, Fig 1; byte-exact, all
 * fields little-endian u32; page_bytes is a power of two):
 *   SP (small page, many vertices with consecutive VIDs):
 *     [rec_0 rec_1 ... rec_{k-1} -> free <- slot_{k-1} ... slot_1 slot_0 | footer]
 *     footer   (last 8 B)         : u32 nslots, u32 kind (= GTS_PAGE_SP)
 *     slot_i   at page_bytes - 8 - 8(i+1): u32 VID, u32 OFF
 *              VID = START_VID + i (VIDs consecutive within a page)
 *     rec_i    at OFF (records are packed in VID order from offset 0):
 *              u32 ADJLIST_SZ, u32 ADJLIST[ADJLIST_SZ]              (unweighted)
 *              u32 ADJLIST_SZ, u32 0, (u32 ADJ, u32 W)[ADJLIST_SZ]  (weighted: every
 *              record 8-byte aligned, an edge's neighbour and weight adjacent, so
 *              one 8-byte load reads both; the weights are not in the paper's
 *              format, R11)
 *   LP (large page: one chunk of the adjacency list of one high-degree
 *       vertex, Fig 1c):
 *     footer   (last 16 B)        : u32 total_deg, u32 chunk_idx,
 *                                   u32 nslots (= 1), u32 kind (= GTS_PAGE_LP)
 *     slot_0   at page_bytes - 16 - 8 : u32 VID, u32 OFF (= 0)
 *     rec_0    at 0               : u32 chunk_len, u32 ADJLIST[chunk_len]
 *                                   (weighted: u32 chunk_len, u32 0, (ADJ, W)[chunk_len])
 *   ADJLIST entries: GTS_ENTRY_VID32 (default) stores the neighbour VID;
 *   GTS_ENTRY_PID16_SLOT16 stores the paper's physical record ID
 *   (ADJ_PID << 16 | ADJ_OFF), whose VID is RVT[ADJ_PID].START_VID + ADJ_OFF
 *   (App A).  Both carry the same information (R-PID in DESIGN.md).
 *   Unused bytes are zero.  SP and LP pages share one page-ID space in VID
 *   order; a vertex is an LP vertex iff its record (4 + 4 deg, weighted 8 + 8 deg)
 *   + its 8-byte slot does not fit an empty SP (R15); greedy packing in VID
 *   order (R15).
 */
#ifndef GTS_H
#define GTS_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define GTS_VERSION 10000 /* 1.0.0 */

typedef enum {
    GTS_OK = 0,
    GTS_EINVAL = -1,        /* bad argument: NULL, src >= n, row_ptr not monotone, col >= n, bad page size */
    GTS_ENOMEM = -2,        /* host or device allocation failed */
    GTS_ECUDA = -3,         /* CUDA runtime error or no usable device */
    GTS_ENCCL = -4,         /* NCCL error (world_size > 1) */
    GTS_EUNSUPPORTED = -5,  /* valid but unsupported combination (e.g. SSSP on an unweighted graph) */
    GTS_EOVERFLOW = -6      /* n >= 2^32, a degree >= 2^32, SSSP distance >= 2^32-1, PID16 limits */
} gts_status;

enum { GTS_PAGE_SP = 0, GTS_PAGE_LP = 1 };
enum { GTS_ENTRY_VID32 = 0, GTS_ENTRY_PID16_SLOT16 = 1 };
/* Strategy-P: pages partitioned h(j) = j mod N, WA replicated, merged after
 *             every iteration / level: PageRank all-reduce(sum),
 *             BFS all-gather + OR of the next frontiers, SSSP all-reduce(min)
 *             + OR, WCC all-reduce(min) of the union-find forests.
 * Strategy-S: WA range-partitioned into N contiguous VID ranges cut at page
 *             boundaries; each rank holds the pages whose sources lie in its
 *             range and routes updates for other ranges to their owners
 *             (north_star "routes updates"): PageRank (dst, value), BFS dst,
 *             SSSP (dst, dist), WCC (dst, label) on GTS_BUILD_SYMMETRIC pages.
 *             Each rank allocates its WA range only (n/N entries).
 * Strategy-S_BCAST: the paper-literal Strategy-S: every rank
 *             processes every page and applies only the updates of its own WA
 *             range (PageRank, BFS, SSSP; WA ranges re-broadcast after each
 *             step); WCC runs the full union-find on every rank (replicated). */
enum { GTS_STRATEGY_P = 0, GTS_STRATEGY_S = 1, GTS_STRATEGY_S_BCAST = 2 };
enum { GTS_RESIDENCY_AUTO = 0, GTS_RESIDENT = 1, GTS_STREAMED = 2 };
enum { GTS_DANGLING_UNIFORM = 0, GTS_DANGLING_DROP = 1 };
enum { GTS_OUT_HOST = 0, GTS_OUT_DEVICE = 1 };
enum { GTS_RUN_TIMING = 1u };   /* gts_run_config.flags: time the main kernels with CUDA events */
/* gts_run_config.flags: Strategy-S routes its remote updates by atomics straight
 * into the owner's WA over peer memory (NVLink / NVSwitch; CUDA IPC mappings
 * between the ranks' processes), fusing the sweep with the exchange: no message
 * buffers, counts or send/recv -- one kernel does the compute and the
 * "collective" (PageRank atomicAdd into the owner's acc, BFS atomicOr into its
 * visited / next bitmaps, SSSP / WCC atomicMin into its dist / labels).  The
 * owners' WA buffers that receive updates while they are read are
 * double-buffered by iteration / level.  Default off (routed messages over
 * NCCL).  Virtual ranks map the other ranks' buffers on the same GPU. */
enum { GTS_ROUTE_PEER = 2u };
/* gts_run_config.flags bits 8-10: the micro-level technique applied inside each
 * slotted page (App E, Fig 14), for gts_bfs and
 * gts_pagerank (other calls reject a non-default value with EUNSUPPORTED).
 *   DEFAULT: the B200 tile engine (BFS) / the hot-set scatter (PageRank);
 *   EDGE:    edge-centric = VWC, a warp per vertex (the paper's default, Alg 2/4);
 *   VERTEX:  vertex-centric, a thread per vertex and all of its edges;
 *   HYBRID:  per page, vertex-centric if the page has < 8 edges per vertex, else
 *            edge-centric (env GTS_HYBRID_DEG overrides the 8);
 *   TILE:    PageRank only: the tile engine with one plain red.add per edge (no hot set).
 * Results are identical for every technique (PageRank: within the fp32 gates). */
enum { GTS_MICRO_DEFAULT = 0u, GTS_MICRO_EDGE = 1u << 8, GTS_MICRO_VERTEX = 2u << 8,
       GTS_MICRO_HYBRID = 3u << 8, GTS_MICRO_TILE = 4u << 8, GTS_MICRO_MASK = 7u << 8 };
/* gts_page_config.flags: store vertices in descending in-degree order (ties by
 * VID) inside the pages.  A builder policy, not a different graph: every call
 * maps its source vertex in and its result out, so callers always see their
 * own VIDs.  The directory and page bytes of such a graph hold the internal
 * IDs (gts_graph_order gives the mapping).  Used by the B200 PageRank kernel
 * to keep the most-updated WA entries contiguous. */
enum { GTS_BUILD_DEGREE_ORDER = 1u };
/* gts_page_config.flags: also store every edge reversed (the pages hold the
 * symmetrised multigraph, 2m entries).  gts_wcc under GTS_STRATEGY_S needs it:
 * its routed label propagation pushes along both directions of an edge from
 * the source's owner only (WCC caveat). */
enum { GTS_BUILD_SYMMETRIC = 2u };
/* gts_page_config.flags: build (and hold in host memory) only the pages that
 * rank owner_rank of an owner_world-rank job processes under owner_strategy
 * (Strategy-P: page j with j mod N == rank; Strategy-S: the rank's
 * contiguous page range).  The directory (RVT) still covers every
 * page.  Such a graph can only be used by a context of that rank and world
 * with that strategy (EINVAL otherwise); gts_graph_pages returns the held
 * pages in ascending page ID.  S_BCAST ranks process every page, so the
 * filter keeps all pages for it. */
enum { GTS_BUILD_OWNER_FILTER = 4u };
#define GTS_OFF 0xFFFFFFFFu

#define GTS_UNREACHED 0xFFFFFFFFu

const char* gts_last_error(void);
int gts_version(void);

/* ------------------------------------------------------------- graphs --- */

typedef struct {
    uint32_t struct_size;     /* sizeof(gts_page_config); 16 (version 1.0 layout) is accepted */
    uint32_t page_bytes;      /* power of two, 256 B .. 1 GiB; default (0) = 1 MiB (R14) */
    uint32_t entry_encoding;  /* GTS_ENTRY_VID32 (default) | GTS_ENTRY_PID16_SLOT16 */
    uint32_t flags;           /* GTS_BUILD_DEGREE_ORDER | GTS_BUILD_SYMMETRIC | GTS_BUILD_OWNER_FILTER */
    /* GTS_BUILD_OWNER_FILTER only: */
    uint32_t owner_rank, owner_world, owner_strategy;
    uint32_t reserved;
} gts_page_config;

typedef struct {
    uint64_t n, m;
    uint64_t num_pages, n_sp, n_lp, n_lp_vertices;
    uint64_t page_bytes;
    uint64_t topo_bytes;      /* num_pages * page_bytes: bytes that move per full sweep */
    uint64_t used_bytes;      /* records + slots + footers actually used */
    uint64_t max_outdeg;
    uint32_t weighted, entry_encoding;
    uint32_t n_hot;           /* entries in the hot-destination table (PageRank, DESIGN.md K-PR) */
    uint32_t ordered;         /* 1 if built with GTS_BUILD_DEGREE_ORDER */
    uint64_t host_page_bytes; /* page bytes this graph holds in host memory (< topo_bytes with an owner filter) */
    uint32_t symmetric;       /* 1 if built with GTS_BUILD_SYMMETRIC (m counts both directions) */
    int32_t owner_rank;       /* GTS_BUILD_OWNER_FILTER: the rank; -1: every page is held */
    uint32_t owner_world, owner_strategy;
} gts_graph_stats;

typedef struct gts_graph gts_graph;   /* opaque; owns the host pages + directory (RVT) */

/* CSR -> slotted pages.
 * row_ptr: n+1 monotone u64 with row_ptr[0] = 0, row_ptr[n] = m; col_idx: m
 * VIDs < n; weights: m values or NULL (a weighted graph is required by
 * gts_sssp).  cfg may be NULL (defaults).  The graph owns a copy of
 * everything; inputs may be freed on return.  Pure host code (no CUDA call).
 * Errors: EINVAL (bad CSR / config), EOVERFLOW (n >= 2^32, degree >= 2^32,
 * PID16 limits: > 65536 pages or > 65536 slots per page), ENOMEM. */
int gts_build_pages(uint64_t n, uint64_t m, const uint64_t* row_ptr, const uint32_t* col_idx,
                    const uint32_t* weights, const gts_page_config* cfg, gts_graph** out);

/* The page plan only (counts of SP/LP pages and bytes) from the degree
 * sequence, without filling pages.  Same rules as gts_build_pages. */
int gts_plan_pages(uint64_t n, const uint64_t* row_ptr, int weighted, const gts_page_config* cfg,
                   gts_graph_stats* out);

int gts_graph_get_stats(const gts_graph* g, gts_graph_stats* out);
/* Host page bytes: num_pages * page_bytes, page j at offset j * page_bytes.
 * Owned by the graph; valid until gts_graph_free. */
const uint8_t* gts_graph_pages(const gts_graph* g);
/* The page directory (RVT, App A) as arrays of num_pages entries:
 * START_VID, number of slots, kind; lp_first/lp_last = first/last page of
 * the LP run a page belongs to (-1 for SP pages; the LP_RANGE of Fig 12, R16).
 * Any pointer may be NULL. */
int gts_graph_directory(const gts_graph* g, uint32_t* start_vid, uint32_t* nslots, uint32_t* kind,
                        int64_t* lp_first, int64_t* lp_last);
/* For a GTS_BUILD_DEGREE_ORDER graph: internal_of[v] = internal ID of caller VID v
 * (n entries).  For other graphs the identity.  EINVAL on NULL. */
int gts_graph_order(const gts_graph* g, uint32_t* internal_of);
void gts_graph_free(gts_graph* g);

/* ------------------------------------------------------------ contexts --- */

typedef struct gts_context gts_context;  /* opaque: device, streams, events, NCCL comm, device buffers */

/* NCCL unique id (128 bytes) created on rank 0 and broadcast by the caller's
 * process group (torch.distributed); needed only when world_size > 1. */
int gts_get_unique_id(uint8_t out[128]);

/* One context per process per GPU (one process per GPU, torchrun style).
 * world_size == 1: unique_id may be NULL and no NCCL is used.
 * world_size > 1 : ranks 0..world_size-1 each call this collectively with the
 * same unique_id; the ranks then run the same gts_* calls collectively. */
int gts_context_create(int device, int rank, int world_size, const uint8_t* unique_id,
                       gts_context** out);
void gts_context_free(gts_context* ctx);
/* Drop the device copy of g's pages (resident pages are cached per graph so
 * their one-time upload stays out of timed runs, as the paper excludes
 * loading). */
int gts_context_evict(gts_context* ctx, const gts_graph* g);
/* Launch on this cudaStream_t (e.g. torch.cuda.current_stream().cuda_stream)
 * instead of the context's own compute stream; NULL restores the default. */
int gts_context_set_stream(gts_context* ctx, void* cuda_stream);

typedef struct {
    uint32_t struct_size;     /* sizeof(gts_run_config) */
    uint32_t strategy;        /* GTS_STRATEGY_P | GTS_STRATEGY_S | GTS_STRATEGY_S_BCAST (see above) */
    uint32_t residency;       /* GTS_RESIDENCY_AUTO | GTS_RESIDENT | GTS_STREAMED */
    uint32_t ring_slots;      /* streamed: device ring depth (0 -> 4) */
    uint32_t batch_pages;     /* streamed: pages per H2D batch (0 -> 64 MiB worth of pages) */
    uint32_t out_location;    /* GTS_OUT_HOST (default) | GTS_OUT_DEVICE (out pointer is device memory on this rank's GPU) */
    uint32_t flags;           /* GTS_RUN_TIMING | one GTS_MICRO_* value */
    uint32_t cache_mib;       /* streamed BFS/SSSP: device LRU cache of topology pages across levels,
                                 in MiB (cachedPIDMap, Alg 1 lines 8/16/29); 0 = none */
    /* ---- version 1.1 (struct_size >= 64; a 32-byte 1.0 config gets the defaults) ---- */
    uint32_t virtual_ranks;   /* 0/1 = off.  V in [2, 8] on a world-1 context: run the V-rank job of
                                 `strategy` on this one GPU -- every rank's page set, WA buffers, kernels
                                 and merge kernels as on V GPUs, the collectives done in device memory
                                 (DESIGN.md "Virtual ranks").  Results equal the real V-rank job's. */
    uint32_t sssp_delta;      /* SSSP near-far bucket width; 0 = unbounded (frontier Bellman-Ford) */
    uint32_t levels_per_sync; /* BFS on one rank, resident: levels enqueued per host round trip; 0 = 8 */
    uint32_t l2_persist_mib;  /* persisting-L2 window on the probed head of WA; 0 = 96 MiB, GTS_OFF = none */
    uint32_t bfs_level_slots; /* BFS level-slot store (one bitmap per level); 0 = 32, GTS_OFF = off */
    uint32_t wcc_sample;      /* WCC sampling pass: first k out-neighbours; 0 = 1, GTS_OFF = no pass */
    uint32_t hybrid_deg;      /* GTS_MICRO_HYBRID: vertex-centric below this many edges/vertex; 0 = 8 */
    uint32_t reserved;
} gts_run_config;

typedef struct {
    double wall_s;            /* host wall clock of the call */
    double upload_s;          /* one-time resident upload inside this call (0 if cached) */
    double main_kernel_s;     /* GTS_RUN_TIMING: summed event time of the expansion/scatter kernels */
    double finish_s;          /* GTS_RUN_TIMING: summed event time of the finish kernels */
    double merge_s;           /* GTS_RUN_TIMING: summed event time of NCCL merges */
    double h2d_s;             /* streamed: summed event time of page copies */
    uint64_t h2d_bytes;       /* topology bytes copied host->device inside the call */
    uint64_t nccl_bytes;      /* bytes this rank contributed to NCCL merges */
    uint64_t pages_processed; /* page visits summed over levels / iterations */
    uint64_t edges_traversed; /* sum of out-degrees of expanded vertices (BFS: reached vertices) */
    uint64_t launches;        /* kernels launched by the library in the call */
    uint64_t main_kernel_launches;
    uint32_t levels_or_iters;
    uint32_t reserved;
    uint64_t cache_hits;      /* streamed + cache: page visits served from the device cache */
    uint64_t cache_misses;    /* streamed + cache: page visits copied from host memory */
    uint64_t wa_bytes;        /* device bytes of the attribute vectors (WA + RA) one rank allocated */
    uint64_t routed_msgs;     /* Strategy-S: update messages sent to other ranks */
} gts_run_stats;

/* BFS (App B.1, Alg 2/3 P:1494-1514; Alg 1 BFS-like path P:330-334).
 * level_out[n]: hop level from src over out-edges, GTS_UNREACHED if not
 * reached (R6, R7).  Bit-exact vs the oracle.  stats may be NULL. */
int gts_bfs(gts_context* ctx, const gts_graph* g, uint64_t src, const gts_run_config* cfg,
            uint32_t* level_out, gts_run_stats* stats);

/* PageRank (App B.2, Alg 4/5 P:1540-1558).
 * x^0 = 1/n; x^t_v = (1-d)/n + d*(sum_{u->v} x^{t-1}_u/outdeg(u) + D/n) with D the
 * dangling mass (UNIFORM, R3) or without it (DROP, paper-literal).  fp32
 * values, fp64 dangling sum.  rank_out[n] fp32. */
int gts_pagerank(gts_context* ctx, const gts_graph* g, uint32_t iters, double damping,
                 uint32_t dangling, const gts_run_config* cfg, float* rank_out, gts_run_stats* stats);

/* SSSP (BFS-like; R11): dist_out[n] u32, GTS_UNREACHED if not
 * reached.  EUNSUPPORTED if g has no weights; EOVERFLOW if a distance would
 * reach 2^32-1. */
int gts_sssp(gts_context* ctx, const gts_graph* g, uint64_t src, const gts_run_config* cfg,
             uint32_t* dist_out, gts_run_stats* stats);

/* WCC ("connected components", PageRank-like; R12):
 * label_out[n] = min VID of v's weakly connected component. */
int gts_wcc(gts_context* ctx, const gts_graph* g, const gts_run_config* cfg, uint32_t* label_out,
            gts_run_stats* stats);

/* Betweenness centrality (BC is run on GTS in the
 * paper, Fig 13c, no kernel given): Brandes' dependency accumulation
 * from each of the k sources over out-edges, unweighted, path counts with
 * edge multiplicity, summed over the sources: bc_out[n] fp64 (not
 * normalised).  Pages may be resident or streamed.  One GPU (EUNSUPPORTED for
 * world_size > 1).  EINVAL if a source >= n. */
int gts_bc(gts_context* ctx, const gts_graph* g, const uint64_t* sources, uint32_t num_sources,
           const gts_run_config* cfg, double* bc_out, gts_run_stats* stats);

/* ---------------------------------------------------- multi-GPU helpers --- */

/* Page -> rank assignment used by a strategy (pure host logic, exposed for
 * tests): owner[num_pages] gets the rank that processes each page, and for
 * GTS_STRATEGY_S vrange[world_size+1] the VID ranges of the WA partition
 * (rank r owns [vrange[r], vrange[r+1])).  vrange may be NULL for P. */
int gts_partition_pages(const gts_graph* g, uint32_t strategy, int world_size, int32_t* owner,
                        uint64_t* vrange);

#ifdef __cplusplus
}
#endif

#endif /* GTS_H */
