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

__device__ __forceinline__ int bits_for(int64_t nvalues) {
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
