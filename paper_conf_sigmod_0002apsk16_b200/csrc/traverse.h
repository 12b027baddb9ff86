// BFS-like drivers shared between translation units (traverse.cu, wcc.cu).
#pragma once

#include "comm.h"

namespace gts {

enum { kBFS = 0, kSSSP = 1, kWCCLP = 2 };   // kWCCLP: routed min-label propagation (WCC under Strategy-S)

int traverse_multi(gts_context* c, const gts_graph* g, uint64_t src, const gts_run_config& rc, Ranks& R, void* out,
                   gts_run_stats* st, int algo, double t_start, bool streamed, double upload_s);

}  // namespace gts
