// exchange.h — multi-GPU plumbing of libshingle.
#pragma once

#include "sg_internal.cuh"

namespace sg {

Exchange *exchange_create(sg_graph *g, const sg_dist *dist);
void exchange_destroy(Exchange *x);
// Pass rows: sums the local row count over ranks and sets the rank's base
// (level 0: n_e and row base; level 1: |S1'| and the canonical k0).
void exchange_row_counts(sg_graph *g, int level, int64_t local_rows);
// Route the pass's pairs to their owner ranks and group them there.
void exchange_and_group(sg_graph *g, int level);
int64_t exchange_sum(sg_graph *g, int64_t v);
void exchange_require_single(sg_graph *g, const char *what);

}  // namespace sg
