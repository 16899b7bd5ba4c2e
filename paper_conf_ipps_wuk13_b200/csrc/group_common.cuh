// group_common.cuh — helpers shared by the grouping kernels (kernels_group.cu,
// kernels_local.cu).
#pragma once

#include <stdint.h>

#include "kernels.h"

namespace sg {
namespace grp {

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

// Bitonic sort, all-ascending ("flip") form, of the index list pm[0, m) by
// (K, V); positions >= m act as +infinity.  Executed by `nthr` threads with
// index `tid`; `sync` is the barrier between steps.  Power-of-two index math.
template <typename IDX, typename KA, typename VA, typename SYNC>
__device__ __forceinline__ void bitonic_idx(IDX *pm, int m, const KA &K, const VA &V, int tid,
                                            int nthr, SYNC sync) {
  int M = 1;
  while (M < m) M <<= 1;
  for (int k = 2; k <= M; k <<= 1) {
    for (int jj = k >> 1; jj > 0; jj >>= 1) {
      for (int t = tid; t < (M >> 1); t += nthr) {
        const int i = ((t & ~(jj - 1)) << 1) | (t & (jj - 1));
        const int l = (jj == (k >> 1)) ? (i ^ (k - 1)) : (i + jj);
        if (l < m) {
          const IDX a = pm[i], b = pm[l];
          if (pair_less(K[b], V[b], K[a], V[a])) {
            pm[i] = b;
            pm[l] = a;
          }
        }
      }
      sync();
    }
  }
}

}  // namespace grp
}  // namespace sg
