// group_common.cuh — helpers shared by the grouping kernels (kernels_group.cu,
// kernels_local.cu).
#pragma once

#include <stdint.h>

#include "kernels.h"

namespace sg {
namespace grp {

// Lanes of the warp (within vm) whose value v agrees with this lane's on the
// low `nbits` bits: the peer mask of __match_any_sync built from nbits
// ballots (short-latency VOTEs instead of one long-latency MATCH; ncu showed
// the MATCH results at the head of the stall chains of the split and local
// sorts).  Every lane of the warp must call it (converged).
__device__ __forceinline__ uint32_t peers_by_ballot(uint32_t v, uint32_t vm, int nbits) {
  uint32_t m = vm;
#pragma unroll
  for (int i = 0; i < 16; ++i) {
    if (i >= nbits) break;
    const uint32_t bit = (v >> i) & 1u;
    const uint32_t b = __ballot_sync(0xffffffffu, bit);
    m &= bit ? b : ~b;
  }
  return m;
}

__host__ __device__ constexpr int bits_for(int64_t nvalues) {
  int b = 0;
  while (((int64_t)1 << b) < nvalues) ++b;
  return b;
}

__device__ __forceinline__ uint32_t top_bits(uint64_t key, int bits) {
  return bits ? (uint32_t)(key >> (64 - bits)) : 0u;
}

// (key, member) is a strict total order within a trial: members are unique.
__device__ __forceinline__ bool pair_less(uint64_t ka, uint32_t va, uint64_t kb, uint32_t vb) {
  return ka < kb || (ka == kb && va < vb);
}

// Final bucket q = (trial j, top `bits` key bits): its pairs sit at
// [sbase, sbase + n) of the final scratch; output position = seg[0] + sbase.
__device__ __forceinline__ void bucket_extent(const GroupArgs &g, int64_t q, int64_t &sbase,
                                              int64_t &n) {
  const int64_t nb = g.plan.nbins;
  const int j = (int)(q / nb);
  n = g.bsize[q];
  sbase = (g.plan.seg[j] - g.plan.seg[0]) + g.bstart[q];
}

}  // namespace grp
}  // namespace sg
