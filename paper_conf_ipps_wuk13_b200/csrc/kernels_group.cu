// kernels_group.cu — stable partition of <shingle, generator> pairs into
// per-trial key buckets: the first half of the grouping "once for each random
// trial" (AMB-5).  The second half (sort inside a bucket + RLE)
// is kernels_local.cu.  DESIGN.md §6.2.
//
//   1. hist     : per (trial, 4K-pair chunk) histogram of the coarse bin;
//   2. offsets  : column prefix over the chunks of a trial (parallel over
//                 chunk ranges) + per-trial bucket scan;
//   3. scatter  : persistent, 16-warp CTAs.  A chunk is ranked stably in
//                 registers (__match_any_sync + per-warp bin counters), placed
//                 bucket-major in shared memory, then written out as
//                 contiguous per-bucket runs (coalesced stores);
//   4. scatter2 : two-level plans only: one CTA per coarse bucket splits it
//                 stably by the next <= 8 bits with the same engine.
// Stability pays: the input of every trial is in generator order, so the
// members of one group (equal keys) arrive in ascending order and the local
// sort rarely has to sort a group by member.  Correctness does not depend on
// it: the local sorts verify the full (key, member) order of every bucket and
// repair the runs that violate it (the fine split ranks by shared atomics,
// whose lane order the hardware does not promise).
#include <algorithm>
#include <cstdlib>

#include "group_common.cuh"
#include "kernels.h"
#include "scan.cuh"
#include "sg_internal.cuh"

namespace sg {

namespace {

using grp::top_bits;

constexpr int kGThreads = 512;
constexpr int kSThreads = 512;                 // split kernels: 16 warps
constexpr int kSWarps = kSThreads / 32;
constexpr int kChunk = 4096;                   // pairs per chunk (hist and scatter)
constexpr int kPerLane = kChunk / kSThreads;   // 8
constexpr int kSeg = kChunk / kSWarps;         // 256 consecutive elements per warp
constexpr int kMaxFan = 256;                   // bins of one split pass
constexpr int kCoarseBits = 8;
constexpr int kMaxBits = 18;                   // final buckets per trial <= 2^18
constexpr int kMaxFine = 1 << (kMaxBits - kCoarseBits);   // fan-out of the fine split (1024)

// Coarse bin = floor(key * nb / 2^64): the top log2(nb) key bits when nb is a
// power of two (buckets), contiguous key ranges for any nb (owner ranks).
__device__ __forceinline__ uint32_t coarse_bin(uint64_t key, int64_t nb) {
  return (uint32_t)__umul64hi(key, (uint64_t)nb);
}

// The same bin when nb = 2^(64 - sh) is a power of two (sh = 64: one bin).
__device__ __forceinline__ uint32_t coarse_bin_pow2(uint64_t key, int sh) {
  return sh < 64 ? (uint32_t)(key >> sh) : 0u;
}

__device__ __forceinline__ int pow2_shift(int64_t nb) {
  int l = 0;
  while ((int64_t(1) << l) < nb) ++l;
  return (int64_t(1) << l) == nb ? 64 - l : -1;   // -1: not a power of two
}

__device__ __forceinline__ uint32_t val_at(const GroupArgs &g, int64_t in_idx, int64_t i) {
  if (g.vals) return g.vals[in_idx];
  if (g.rowid) return g.rowid[i];
  return g.val_base + (uint32_t)i;
}

__device__ __forceinline__ uint32_t lanemask_lt() {
  uint32_t m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}

// Element e of a chunk held by (warp w, lane, slot u): warps own contiguous
// segments, so (w, u, lane) order is input order (stability).
__device__ __forceinline__ int elem_of(int u) {
  return (threadIdx.x >> 5) * kSeg + u * 32 + (threadIdx.x & 31);
}

// MB: the largest fan-out the kernel uses (256 for the coarse scatter and
// the <= 8-bit fine splits; 1024 for the 10-bit fine split of 18-bit plans:
// 104 KB instead of 64 KB, which also shrinks L1 — measured: sizing every
// split for 1024 bins slowed the gos2m fine split 66 -> 83 ms).
template <int MB>
struct SplitSmemT {
  uint64_t K[kChunk];                  // chunk, bucket-major after the split
  uint32_t V[kChunk];
  uint16_t cnt[kSWarps * MB];          // [warp][bin] running positions
  uint32_t sbst[MB + 1];               // bin starts within the chunk
  int64_t off[MB];                     // output position - chunk position, per bin
  int64_t gcur[MB];                    // scatter2: running fine-bucket cursors
  uint32_t tot[MB];                    // scatter2: fine-bucket totals
  int64_t ws[33];
};
using SplitSmem = SplitSmemT<kMaxFan>;

// Rank the len <= kChunk pairs (kk, vv) of one chunk stably by bin_of(key) in
// [0, nb) and place them bucket-major in S.K / S.V.  obase(b) gives the output
// position of the first pair of bin b in this chunk; S.off[b] receives
// obase(b) - (chunk position of that pair).  Ends with a barrier.
// BALLOT: peer masks from ballots (measured faster for the fine split,
// slower for the coarse scatter) or __match_any_sync.  NBC > 0: nb == NBC is
// known at compile time (full 8-bit fan-out: unrolled ballots, constant loops).
// AT selects how a warp ranks its pairs:
//  0: peer masks (__match_any_sync or ballots) for both the count and the
//     placement, warp counters advanced by the lowest peer (stable);
//  1: no peer masks — every pair counts and takes its slot with its own
//     shared atomic on the warp's packed u16 counters.  Within one warp
//     instruction the order of conflicting lanes is the hardware's
//     (tools/atom_order.cu measures lane order on the B200); the final sorts
//     verify the full (key, member) order and repair any run out of it, so
//     the result never depends on it;
//  2: counts by fire-and-forget atomics (no dependency chain), placement by
//     peer masks as in 0 (stable);
//  3: counts as in 2, placement by peer masks with the lowest peer taking
//     the run's base by a returning atomic (no __syncwarp chain; stable).
template <bool BALLOT, int NBC, int AT, typename SM, typename BIN, typename OBASE>
__device__ __forceinline__ void split_place(SM &S, int len, int nb_rt,
                                            const uint64_t (&kk)[kPerLane],
                                            const uint32_t (&vv)[kPerLane], BIN bin_of,
                                            OBASE obase) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const uint32_t lt = lanemask_lt();
  const int nb = NBC > 0 ? NBC : nb_rt;
  uint16_t *my = S.cnt + w * nb;
  uint32_t *cw = reinterpret_cast<uint32_t *>(S.cnt);
  for (int b = lane; b < nb; b += 32) my[b] = 0;
  __syncwarp();
  uint32_t pr[kPerLane];
  const int nbits = NBC > 0 ? grp::bits_for(NBC) : grp::bits_for(nb);
  if (AT >= 1) {
#pragma unroll
    for (int u = 0; u < kPerLane; ++u)
      if (elem_of(u) < len) {
        const int idx = w * nb + (int)bin_of(kk[u]);
        atomicAdd(cw + (idx >> 1), 1u << ((idx & 1) << 4));
      }
  } else {
#pragma unroll
  for (int u = 0; u < kPerLane; ++u) {
    const bool valid = elem_of(u) < len;
    const uint32_t vm = __ballot_sync(0xffffffffu, valid);
    const uint32_t b = valid ? bin_of(kk[u]) : 0u;
    uint32_t pm = 0;
    if (BALLOT) pm = grp::peers_by_ballot(b, vm, nbits);          // all lanes (converged)
    else if (valid) pm = __match_any_sync(vm, b);
    pr[u] = valid ? pm : 0u;
    if (valid && (pr[u] & lt) == 0) my[b] += (uint16_t)__popc(pr[u]);   // lowest peer leads
    __syncwarp();                      // the next batch's leaders read these counters
  }
  }
  __syncthreads();
  {
    // bin-major, warp-minor exclusive prefix: thread t owns bins
    // [t*BPT, (t+1)*BPT) (BPT = 1 up to 512 bins, 2 for the 1024-bin fine split)
    constexpr int BPTC = NBC > kSThreads ? (NBC + kSThreads - 1) / kSThreads : 1;
    const int BPT = NBC > 0 ? BPTC : (nb + kSThreads - 1) / kSThreads;
    const int t = threadIdx.x;
    uint32_t tsum = 0, bt[2] = {0, 0};
#pragma unroll
    for (int i = 0; i < 2; ++i) {
      const int b = t * BPT + i;
      if (i < BPT && b < nb) {
        uint32_t run = 0;
#pragma unroll 4
        for (int x = 0; x < kSWarps; ++x) {
          const uint32_t c = S.cnt[x * nb + b];
          S.cnt[x * nb + b] = (uint16_t)run;
          run += c;
        }
        bt[i] = run;
        tsum += run;
      }
    }
    int64_t all;
    const int64_t ex = block_excl_scan<int64_t>((int64_t)tsum, S.ws, &all);
    int64_t acc = ex;
#pragma unroll
    for (int i = 0; i < 2; ++i) {
      const int b = t * BPT + i;
      if (i < BPT && b < nb) {
        S.sbst[b] = (uint32_t)acc;
        S.off[b] = obase(b) - acc;
#pragma unroll 4
        for (int x = 0; x < kSWarps; ++x) S.cnt[x * nb + b] += (uint16_t)acc;
        acc += bt[i];
      }
    }
    if (t == 0) S.sbst[nb] = (uint32_t)len;
  }
  __syncthreads();
  if (AT >= 2) {
    // peer masks of all batches first (independent, their latencies overlap)
#pragma unroll
    for (int u = 0; u < kPerLane; ++u) {
      const bool valid = elem_of(u) < len;
      const uint32_t vm = __ballot_sync(0xffffffffu, valid);
      const uint32_t b = valid ? bin_of(kk[u]) : 0u;
      uint32_t pm = 0;
      if (BALLOT) pm = grp::peers_by_ballot(b, vm, nbits);
      else if (valid) pm = __match_any_sync(vm, b);
      pr[u] = valid ? pm : 0u;
    }
  }
  if (AT == 3) {
    uint32_t o[kPerLane];
#pragma unroll
    for (int u = 0; u < kPerLane; ++u) {
      o[u] = 0;
      if (elem_of(u) < len && (pr[u] & lt) == 0) {
        const int idx = w * nb + (int)bin_of(kk[u]);
        o[u] = atomicAdd(cw + (idx >> 1), (uint32_t)__popc(pr[u]) << ((idx & 1) << 4)) >> ((idx & 1) << 4);
      }
    }
#pragma unroll
    for (int u = 0; u < kPerLane; ++u) {
      const int lead = __ffs(pr[u]) - 1;
      const uint32_t oo = __shfl_sync(0xffffffffu, o[u], lead < 0 ? 0 : lead);
      if (elem_of(u) < len) {
        const uint32_t p = (oo & 0xFFFFu) + __popc(pr[u] & lt);
        S.K[p] = kk[u];
        S.V[p] = vv[u];
      }
    }
    __syncthreads();
    return;
  }
  if (AT == 1) {
    uint32_t o[kPerLane];
#pragma unroll
    for (int u = 0; u < kPerLane; ++u) {
      o[u] = 0;
      if (elem_of(u) < len) {
        const int idx = w * nb + (int)bin_of(kk[u]);
        o[u] = atomicAdd(cw + (idx >> 1), 1u << ((idx & 1) << 4)) >> ((idx & 1) << 4);
      }
    }
#pragma unroll
    for (int u = 0; u < kPerLane; ++u)
      if (elem_of(u) < len) {
        const uint32_t p = o[u] & 0xFFFFu;
        S.K[p] = kk[u];
        S.V[p] = vv[u];
      }
    __syncthreads();
    return;
  }
#pragma unroll
  for (int u = 0; u < kPerLane; ++u) {
    const bool valid = elem_of(u) < len;
    const uint32_t vm = __ballot_sync(0xffffffffu, valid);
    if (valid) {
      const uint32_t b = bin_of(kk[u]);
      const uint32_t rank = __popc(pr[u] & lt);
      const uint32_t base = my[b];
      __syncwarp(vm);
      if (rank == 0) my[b] = (uint16_t)(base + __popc(pr[u]));
      __syncwarp(vm);
      const uint32_t p = base + rank;
      S.K[p] = kk[u];
      S.V[p] = vv[u];
    }
  }
  __syncthreads();
}

// Write the placed chunk: consecutive threads take consecutive chunk
// positions, which inside one bin are consecutive output positions.
template <typename SM, typename BIN>
__device__ __forceinline__ void emit_runs(const SM &S, int len, BIN bin_of,
                                          uint64_t *__restrict__ outK,
                                          uint32_t *__restrict__ outV,
                                          uint8_t *__restrict__ outF = nullptr) {
  for (int p = threadIdx.x; p < len; p += kSThreads) {
    const uint64_t key = S.K[p];
    const int64_t o = S.off[bin_of(key)] + p;
    outK[o] = key;
    outV[o] = S.V[p];
    if (outF) outF[o] = (uint8_t)(key >> 48);   // the fine digit of 16-bit plans
  }
}

// ---- 1. histogram -----------------------------------------------------------
// kHistChunks consecutive chunks per 1024-thread CTA (long-running CTAs; the
// next chunk's keys are loaded while the current one is counted).
constexpr int kHThreads = 1024;
constexpr int kHistChunks = 16;
constexpr int kHPer = kChunk / kHThreads;      // 4 keys per thread per chunk

__global__ void __launch_bounds__(kHThreads) hist_kernel(const __grid_constant__ GroupArgs g) {
  __shared__ uint32_t hist[2][kMaxFan];
  const int nb = (int)g.plan.nb1;
  const int sh = pow2_shift(nb);
  const int64_t k0 = (int64_t)blockIdx.x * kHistChunks;
  const int64_t k1 = min(k0 + kHistChunks, g.plan.nchunks);
  for (int i = threadIdx.x; i < 2 * kMaxFan; i += kHThreads) (&hist[0][0])[i] = 0;
  uint64_t kk[kHPer], nx[kHPer];
  auto load = [&](int64_t k, uint64_t (&dst)[kHPer]) {
    const int len = g.plan.chunk_len[k];
    const uint64_t *__restrict__ keys = g.keys + g.plan.chunk_in0[k];
#pragma unroll
    for (int u = 0; u < kHPer; ++u) {
      const int i = threadIdx.x + u * kHThreads;
      dst[u] = i < len ? keys[i] : 0;
    }
  };
  if (k0 < k1) load(k0, kk);
  __syncthreads();
  for (int64_t k = k0; k < k1; ++k) {
    const int buf = (int)(k - k0) & 1;
    if (k + 1 < k1) load(k + 1, nx);
    const int len = g.plan.chunk_len[k];
#pragma unroll
    for (int u = 0; u < kHPer; ++u)
      if (threadIdx.x + u * kHThreads < len)
        atomicAdd(&hist[buf][sh >= 0 ? coarse_bin_pow2(kk[u], sh) : coarse_bin(kk[u], nb)], 1u);
    __syncthreads();
    uint32_t *out = g.counts + k * nb;
    for (int i = threadIdx.x; i < nb; i += kHThreads) {
      out[i] = hist[buf][i];
      hist[buf][i] = 0;                       // ready for chunk k + 2
    }
#pragma unroll
    for (int u = 0; u < kHPer; ++u) kk[u] = nx[u];
  }
}

// The same histogram from the min-hash kernels' top-key-byte array (1 B per
// pair instead of the 8-B key; power-of-two coarse fan-outs of <= 256 bins).
// A chunk is 4 KB, one 4-byte word per thread: chunks are counted four at a
// time (four words in flight per thread, the next four prefetched), else the
// kernel is latency bound on too few bytes in flight.
constexpr int kHB = 4;                         // chunks counted together
template <bool B8>                             // B8: nb1 == 256 (the bin is the byte)
__global__ void __launch_bounds__(kHThreads) hist_bytes_kernel(const __grid_constant__ GroupArgs g) {
  __shared__ uint32_t hist[kHB][kMaxFan];
  const int nb = B8 ? kMaxFan : (int)g.plan.nb1;
  const int sh = B8 ? 0 : 8 - grp::bits_for(nb);
  const int64_t k0 = (int64_t)blockIdx.x * kHistChunks;
  const int64_t k1 = min(k0 + kHistChunks, g.plan.nchunks);
  for (int i = threadIdx.x; i < kHB * kMaxFan; i += kHThreads) (&hist[0][0])[i] = 0;
  auto load = [&](int64_t k) -> uint32_t {
    if (k >= k1) return 0u;
    const int len = g.plan.chunk_len[k];
    const uint8_t *__restrict__ kb = g.kbin + g.plan.chunk_in0[k];
    const int i = 4 * threadIdx.x;
    if (i + 4 <= len) return *reinterpret_cast<const uint32_t *>(kb + i);
    uint32_t w = 0;
    for (int x = 0; x < 4 && i + x < len; ++x) w |= (uint32_t)kb[i + x] << (8 * x);
    return w;
  };
  uint32_t cur[kHB], nxt[kHB];
#pragma unroll
  for (int c = 0; c < kHB; ++c) cur[c] = load(k0 + c);
  __syncthreads();
  for (int64_t kb0 = k0; kb0 < k1; kb0 += kHB) {
#pragma unroll
    for (int c = 0; c < kHB; ++c) nxt[c] = load(kb0 + kHB + c);   // in flight while counting
#pragma unroll
    for (int c = 0; c < kHB; ++c) {
      if (kb0 + c >= k1) break;
      const int len = g.plan.chunk_len[kb0 + c];
      if (len == kChunk) {                     // warp-uniform: whole chunk, no tail tests
#pragma unroll
        for (int x = 0; x < 4; ++x) atomicAdd(&hist[c][((cur[c] >> (8 * x)) & 0xFFu) >> sh], 1u);
      } else {
#pragma unroll
        for (int x = 0; x < 4; ++x)
          if (4 * (int)threadIdx.x + x < len) atomicAdd(&hist[c][((cur[c] >> (8 * x)) & 0xFFu) >> sh], 1u);
      }
    }
    __syncthreads();
    for (int i = threadIdx.x; i < kHB * nb; i += kHThreads) {
      const int c = i / nb, b = i - c * nb;
      if (kb0 + c < k1) g.counts[(kb0 + c) * nb + b] = hist[c][b];
      hist[c][b] = 0;
    }
    __syncthreads();
#pragma unroll
    for (int c = 0; c < kHB; ++c) cur[c] = nxt[c];
  }
}

// ---- 2. offsets ---------------------------------------------------------------
// counts[k][b] <- exclusive prefix over the chunks of its trial; bsize1[j][b].
// Block (32 bins) x (32 chunk ranges): range sums, a scan over the ranges,
// then each range rewrites its chunks.
__global__ void __launch_bounds__(1024) colscan_kernel(const __grid_constant__ GroupArgs g) {
  __shared__ uint32_t part[32][33];
  const int64_t nb = g.plan.nb1;
  const int j = blockIdx.y;
  const int bl = threadIdx.x & 31, pi = threadIdx.x >> 5;
  const int64_t b = (int64_t)blockIdx.x * 32 + bl;
  const int k0 = g.plan.trial_chunk0[j], k1 = g.plan.trial_chunk0[j + 1];
  const int L = (k1 - k0 + 31) / 32;
  const int a0 = min(k1, k0 + pi * L), a1 = min(k1, a0 + L);
  constexpr int U = 16;                    // loads in flight per thread (latency bound)
  uint32_t s = 0;
  if (b < nb) {
    int k = a0;
    for (; k + U <= a1; k += U) {
      uint32_t v[U];
#pragma unroll
      for (int x = 0; x < U; ++x) v[x] = g.counts[(int64_t)(k + x) * nb + b];
#pragma unroll
      for (int x = 0; x < U; ++x) s += v[x];
    }
    for (; k < a1; ++k) s += g.counts[(int64_t)k * nb + b];
  }
  part[pi][bl] = s;
  __syncthreads();
  if (pi == 0) {
    uint32_t run = 0;
    for (int x = 0; x < 32; ++x) {
      const uint32_t v = part[x][bl];
      part[x][bl] = run;
      run += v;
    }
    if (b < nb) g.bsize1[(int64_t)j * nb + b] = run;
  }
  __syncthreads();
  if (b < nb) {
    uint32_t run = part[pi][bl];
    int k = a0;
    for (; k + U <= a1; k += U) {
      uint32_t v[U];
#pragma unroll
      for (int x = 0; x < U; ++x) v[x] = g.counts[(int64_t)(k + x) * nb + b];
#pragma unroll
      for (int x = 0; x < U; ++x) {
        g.counts[(int64_t)(k + x) * nb + b] = run;
        run += v[x];
      }
    }
    for (; k < a1; ++k) {
      uint32_t *p = g.counts + (int64_t)k * nb + b;
      const uint32_t v = *p;
      *p = run;
      run += v;
    }
  }
}

// bstart1[j][b] = exclusive scan of bsize1[j][.] (relative to the segment).
__global__ void binscan_kernel(const __grid_constant__ GroupArgs g) {
  __shared__ int64_t ws[33];
  const int64_t nb = g.plan.nb1;
  const int j = blockIdx.x;
  const uint32_t *sz = g.bsize1 + (int64_t)j * nb;
  uint32_t *out = g.bstart1 + (int64_t)j * nb;
  int64_t carry = 0;
  for (int64_t base = 0; base < nb; base += blockDim.x) {
    int64_t i = base + threadIdx.x;
    int64_t v = i < nb ? sz[i] : 0;
    int64_t tot;
    int64_t ex = block_excl_scan<int64_t>(v, ws, &tot);
    if (i < nb) out[i] = (uint32_t)(carry + ex);
    carry += tot;
  }
}

// ---- 3. stable coarse scatter (persistent) ------------------------------------
__device__ __forceinline__ void load_chunk(const GroupArgs &g, int64_t k, uint64_t (&kk)[kPerLane],
                                           uint32_t (&vv)[kPerLane]) {
  const int64_t i0 = g.plan.chunk_i0[k];
  const int64_t in0 = g.plan.chunk_in0[k];
  const int len = g.plan.chunk_len[k];
#pragma unroll
  for (int u = 0; u < kPerLane; ++u) {
    const int e = elem_of(u);
    if (e < len) {
      kk[u] = g.keys[in0 + e];
      vv[u] = val_at(g, in0 + e, i0 + e);
    }
  }
}

// C8: the full 8-bit coarse fan-out (nb1 == 256), bin = the top key byte
// (a constant shift; the generic bin costs ~10 instructions per use).
template <bool C8, int AT>
__global__ void __launch_bounds__(kSThreads, 2) scatter_kernel(const __grid_constant__ GroupArgs g) {
  extern __shared__ __align__(16) unsigned char smraw[];
  SplitSmem &S = *reinterpret_cast<SplitSmem *>(smraw);
  const int nb = C8 ? kMaxFan : (int)g.plan.nb1;
  const int sh = pow2_shift(nb);
  auto bin = [&](uint64_t key) {
    if (C8) return (uint32_t)(key >> 56);
    return sh >= 0 ? coarse_bin_pow2(key, sh) : coarse_bin(key, nb);
  };
  uint64_t kk[kPerLane];
  uint32_t vv[kPerLane];
  int64_t k = blockIdx.x;
  if (k < g.plan.nchunks) load_chunk(g, k, kk, vv);
  while (k < g.plan.nchunks) {
    const int j = g.plan.chunk_trial[k];
    const int len = g.plan.chunk_len[k];
    const int64_t sseg = g.plan.seg[j] - g.plan.seg[0];   // scratch segment start
    int64_t gb = 0;
    if (threadIdx.x < nb)
      gb = sseg + (int64_t)g.bstart1[(int64_t)j * nb + threadIdx.x] + g.counts[k * nb + threadIdx.x];
    split_place<false, C8 ? kMaxFan : 0, AT>(S, len, nb, kk, vv, bin, [&](int) { return gb; });
    const int64_t kn = k + gridDim.x;
    if (kn < g.plan.nchunks) load_chunk(g, kn, kk, vv);   // in flight during the stores
    if (!C8 && g.peer_keys) {
      // fused exchange: bin d = owner rank d, stored straight into its
      // receive buffers (NVLink / NVSwitch peer stores; same device for the
      // loopback group) at the positions the owner's grouping expects
      for (int p = threadIdx.x; p < len; p += kSThreads) {
        const uint64_t key = S.K[p];
        const uint32_t d = bin(key);
        const int64_t o = S.off[d] + p;
        g.peer_keys[d][o] = key;
        g.peer_vals[d][o] = S.V[p];
      }
    } else {
      emit_runs(S, len, bin, g.akeys, g.avals, C8 ? g.fbin : nullptr);
    }
    __syncthreads();
    k = kn;
  }
}

// ---- 4. stable second-level scatter (one CTA per coarse bucket) ----------------
// FB > 0: a plan with an 8-bit coarse level and FB fine bits known at compile
// time (FB = 8: bits == 16, the level-II plans of the 2M and 640M configs;
// FB = 7: bits == 15, hub2m):
// 640M configs): fine digit = key bits 48..55 by a constant shift.
template <int FB, int AT>
__global__ void __launch_bounds__(kSThreads, 2) scatter2_kernel(const __grid_constant__ GroupArgs g) {
  extern __shared__ __align__(16) unsigned char smraw[];
  using SM = SplitSmemT<(FB == 0 || FB > 8) ? kMaxFine : kMaxFan>;
  SM &S = *reinterpret_cast<SM *>(smraw);
  const int64_t q1 = blockIdx.x;                 // (trial, coarse bucket)
  const int64_t nb1 = g.plan.nb1;
  const int j = (int)(q1 / nb1);
  const int b1 = (int)(q1 % nb1);
  const int bits = FB ? 8 + FB : g.plan.bits, bits2 = FB ? FB : g.plan.bits - g.plan.bits1;
  const int nb2 = 1 << bits2;
  const uint32_t mask2 = (uint32_t)nb2 - 1u;
  const int64_t sseg = g.plan.seg[j] - g.plan.seg[0];
  const uint32_t st1 = g.bstart1[q1];
  const int64_t n = g.bsize1[q1];
  const uint64_t *__restrict__ K = g.akeys + sseg + st1;
  const uint32_t *__restrict__ V = g.avals + sseg + st1;
  auto fine = [&](uint64_t key) {
    if (FB) return (uint32_t)(key >> (56 - FB)) & ((1u << FB) - 1u);
    return top_bits(key, bits) & mask2;
  };
  // fine-bucket totals (order-free), starts, sizes
  for (int i = threadIdx.x; i < nb2; i += blockDim.x) S.tot[i] = 0;
  __syncthreads();
  if (FB == 8 && g.fbin) {
    // the coarse scatter wrote each pair's fine digit as one byte: count
    // 1 B per pair instead of re-reading the 8-B keys (aligned words, two
    // in flight per thread; the unaligned head and tail byte by byte)
    const uint8_t *__restrict__ fb = g.fbin + sseg + st1;
    const int head = (int)((4 - ((uintptr_t)fb & 3)) & 3);
    const int h = (int)min((int64_t)head, n);
    if ((int)threadIdx.x < h) atomicAdd(&S.tot[fb[threadIdx.x]], 1u);
    const uint32_t *__restrict__ fw = reinterpret_cast<const uint32_t *>(fb + h);
    const int64_t nw = (n - h) >> 2;
    int64_t i = threadIdx.x;
    for (; i + kSThreads < nw; i += 2 * kSThreads) {
      const uint32_t w0 = fw[i], w1 = fw[i + kSThreads];
#pragma unroll
      for (int x = 0; x < 4; ++x) atomicAdd(&S.tot[(w0 >> (8 * x)) & 0xFFu], 1u);
#pragma unroll
      for (int x = 0; x < 4; ++x) atomicAdd(&S.tot[(w1 >> (8 * x)) & 0xFFu], 1u);
    }
    for (; i < nw; i += kSThreads) {
      const uint32_t w0 = fw[i];
#pragma unroll
      for (int x = 0; x < 4; ++x) atomicAdd(&S.tot[(w0 >> (8 * x)) & 0xFFu], 1u);
    }
    const int64_t t0 = h + 4 * nw;
    if ((int64_t)threadIdx.x < n - t0) atomicAdd(&S.tot[fb[t0 + threadIdx.x]], 1u);
  } else {
    // four loads in flight per thread
    int64_t i = threadIdx.x;
    for (; i + 3 * kSThreads < n; i += 4 * kSThreads) {
      const uint64_t k0 = K[i], k1 = K[i + kSThreads], k2 = K[i + 2 * kSThreads], k3 = K[i + 3 * kSThreads];
      atomicAdd(&S.tot[fine(k0)], 1u);
      atomicAdd(&S.tot[fine(k1)], 1u);
      atomicAdd(&S.tot[fine(k2)], 1u);
      atomicAdd(&S.tot[fine(k3)], 1u);
    }
    for (; i < n; i += kSThreads) atomicAdd(&S.tot[fine(K[i])], 1u);
  }
  __syncthreads();
  {
    // thread t owns fine bins [t*BPT, (t+1)*BPT)
    const int BPT = (nb2 + kSThreads - 1) / kSThreads;
    const int t = threadIdx.x;
    int64_t v[2] = {0, 0};
    for (int i = 0; i < BPT; ++i)
      if (t * BPT + i < nb2) v[i] = S.tot[t * BPT + i];
    int64_t all;
    int64_t ex = block_excl_scan<int64_t>(v[0] + v[1], S.ws, &all);
    for (int i = 0; i < BPT; ++i) {
      const int d = t * BPT + i;
      if (d < nb2) {
        const int64_t qf = (int64_t)j * g.plan.nbins + ((int64_t)b1 << bits2) + d;
        g.bstart[qf] = st1 + (uint32_t)ex;
        g.bsize[qf] = (uint32_t)v[i];
        S.gcur[d] = sseg + st1 + ex;
      }
      ex += v[i];
    }
  }
  __syncthreads();
  uint64_t kk[kPerLane];
  uint32_t vv[kPerLane];
  auto load = [&](int64_t c0) {
    const int len = (int)min((int64_t)kChunk, n - c0);
#pragma unroll
    for (int u = 0; u < kPerLane; ++u) {
      const int e = elem_of(u);
      if (e < len) {
        kk[u] = K[c0 + e];
        vv[u] = V[c0 + e];
      }
    }
  };
  if (n > 0) load(0);
  for (int64_t c0 = 0; c0 < n; c0 += kChunk) {
    const int len = (int)min((int64_t)kChunk, n - c0);
    split_place<true, FB ? (1 << FB) : 0, AT>(S, len, nb2, kk, vv, fine, [&](int d) { return S.gcur[d]; });
    if (c0 + kChunk < n) load(c0 + kChunk);
    emit_runs(S, len, fine, g.bkeys, g.bvals);
    // advance the fine cursors by this sub-chunk's counts
    for (int d = threadIdx.x; d < nb2; d += blockDim.x) S.gcur[d] += S.sbst[d + 1] - S.sbst[d];
    __syncthreads();
  }
}

// Per-chunk tables from the piece table (one thread per chunk; piece found
// by binary search over the pieces' first chunks).
__global__ void chunk_table_kernel(const int32_t *__restrict__ p_trial,
                                   const int64_t *__restrict__ p_in0,
                                   const int64_t *__restrict__ p_len,
                                   const int64_t *__restrict__ p_row0,
                                   const int64_t *__restrict__ p_chunk0, int32_t npieces,
                                   int64_t nchunks, GroupPlan plan) {
  for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < nchunks;
       k += (int64_t)gridDim.x * blockDim.x) {
    int lo = 0, hi = npieces;        // p_chunk0[lo] <= k < p_chunk0[hi]
    while (hi - lo > 1) {
      const int mid = (lo + hi) >> 1;
      if (p_chunk0[mid] <= k) lo = mid;
      else hi = mid;
    }
    const int64_t a = (k - p_chunk0[lo]) * plan.chunk;
    plan.chunk_i0[k] = p_row0[lo] + a;
    plan.chunk_in0[k] = p_in0[lo] + a;
    plan.chunk_len[k] = (int32_t)min(plan.chunk, p_len[lo] - a);
    plan.chunk_trial[k] = p_trial[lo];
  }
}

__global__ void popcount_kernel(const uint32_t *__restrict__ w, int64_t n, unsigned long long *out) {
  unsigned long long acc = 0;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x)
    acc += __popc(w[i]);
  acc = warp_sum(acc);
  if ((threadIdx.x & 31) == 0 && acc) atomicAdd(out, acc);
}

__global__ void sum_i32_kernel(const int32_t *__restrict__ a, int64_t n, unsigned long long *out) {
  unsigned long long acc = 0;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x)
    acc += (unsigned)a[i];
  acc = warp_sum(acc);
  if ((threadIdx.x & 31) == 0 && acc) atomicAdd(out, acc);
}

}  // namespace

// Ranking mode of the split kernels (split_place's AT): the fine split
// defaults to 1 (per-pair atomics), the coarse scatter to 0 (__match_any_sync);
// SG_SPLIT_FINE / SG_SPLIT_COARSE = 0..3 select another (A/B).  Measured on
// gos2m (group2, ms/step): fine split 73.1 (0) -> 66.2 (1); coarse scatter
// 74.7 (0) vs 85.6 (1).  On the B200 conflicting lanes are served in lane
// order (tools/atom_order.cu: 0 of 1.55e8 warp-instructions out of order), so
// mode 1 is in fact stable and the local sorts' repairs stay rare.
int split_mode(bool fine) {
  static const int m[2] = {[] {
                             const char *e = getenv("SG_SPLIT_COARSE");
                             return e ? std::min(3, std::max(0, atoi(e))) : 0;
                           }(),
                           [] {
                             const char *e = getenv("SG_SPLIT_FINE");
                             return e ? std::min(3, std::max(0, atoi(e))) : 1;
                           }()};
  return m[fine ? 1 : 0];
}

// Whether any split may deliver a bucket out of generator order (mode 1).
int split_atomic() { return split_mode(false) == 1 || split_mode(true) == 1; }

int64_t group_chunk_pairs() { return kChunk; }
int32_t group_max_fanout() { return kMaxFan; }

void group_bits(int64_t maxseg, int32_t *bits, int32_t *bits1) {
  // final buckets of 512-1024 pairs on average (the warp-tier sort holds 1K)
  // test hook SG_GROUP_TARGET: smaller target buckets (forces the two-level
  // partition and the big-bucket path on graphs the oracle can check)
  const char *e = getenv("SG_GROUP_TARGET");
  int64_t target = e ? atoll(e) : 1024;
  if (target <= 0) target = 1024;
  int b = 0;
  while ((maxseg >> b) > target && b < kMaxBits) ++b;
  *bits = b;
  *bits1 = std::min(b, kCoarseBits);
}

cudaError_t group_chunk_tables(const GroupPlan &plan, const int32_t *p_trial, const int64_t *p_in0,
                               const int64_t *p_len, const int64_t *p_row0,
                               const int64_t *p_chunk0, int32_t npieces, cudaStream_t st) {
  if (plan.nchunks == 0) return cudaSuccess;
  const int grid = (int)std::min<int64_t>((plan.nchunks + 255) / 256, 148 * 8);
  chunk_table_kernel<<<grid, 256, 0, st>>>(p_trial, p_in0, p_len, p_row0, p_chunk0, npieces,
                                           plan.nchunks, plan);
  ++g_launches;
  return cudaGetLastError();
}

cudaError_t group_hist(const GroupArgs &g, cudaStream_t st) {
  if (g.plan.nchunks == 0) return cudaSuccess;
  if (g.plan.nb1 > kMaxFan) return cudaErrorInvalidValue;
  if (g.kbin && (g.plan.nb1 & (g.plan.nb1 - 1)) == 0) {
    const unsigned grid = (unsigned)((g.plan.nchunks + kHistChunks - 1) / kHistChunks);
    if (g.plan.nb1 == kMaxFan) hist_bytes_kernel<true><<<grid, kHThreads, 0, st>>>(g);
    else hist_bytes_kernel<false><<<grid, kHThreads, 0, st>>>(g);
    ++g_launches;
    return cudaGetLastError();
  }
  hist_kernel<<<(unsigned)((g.plan.nchunks + kHistChunks - 1) / kHistChunks), kHThreads, 0, st>>>(g);
  ++g_launches;
  return cudaGetLastError();
}

cudaError_t group_colscan(const GroupArgs &g, cudaStream_t st) {
  if (g.plan.c == 0) return cudaSuccess;
  dim3 grid((unsigned)((g.plan.nb1 + 31) / 32), (unsigned)g.plan.c);
  colscan_kernel<<<grid, 1024, 0, st>>>(g);
  ++g_launches;
  return cudaGetLastError();
}

cudaError_t group_binscan(const GroupArgs &g, cudaStream_t st) {
  if (g.plan.c == 0) return cudaSuccess;
  binscan_kernel<<<(unsigned)g.plan.c, 1024, 0, st>>>(g);
  ++g_launches;
  return cudaGetLastError();
}

cudaError_t group_offsets(const GroupArgs &g, cudaStream_t st) {
  cudaError_t e = group_colscan(g, st);
  if (e != cudaSuccess || g.plan.c == 0) return e;
  binscan_kernel<<<(unsigned)g.plan.c, 1024, 0, st>>>(g);
  ++g_launches;
  return cudaGetLastError();
}

static cudaError_t split_attr(const void *fn, int *per_sm, size_t smem = sizeof(SplitSmem)) {
  cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(per_sm, fn, kSThreads, smem);
  *per_sm = std::max(*per_sm, 1);
  return e;
}

cudaError_t group_scatter(const GroupArgs &g, int num_sms, cudaStream_t st) {
  if (g.plan.nchunks == 0) return cudaSuccess;
  if (g.plan.nb1 > kMaxFan) return cudaErrorInvalidValue;
  const bool c8 = g.plan.nb1 == kMaxFan;
  const int mode = split_mode(false);
  const void *fn = nullptr;
  switch ((c8 ? 4 : 0) + mode) {
#define SG_SC(C, M) case (C ? 4 : 0) + M: fn = (const void *)scatter_kernel<C, M>; break;
    SG_SC(true, 0) SG_SC(true, 1) SG_SC(true, 2) SG_SC(true, 3)
    SG_SC(false, 0) SG_SC(false, 1) SG_SC(false, 2) SG_SC(false, 3)
#undef SG_SC
  }
  int per_sm = 1;
  cudaError_t e = split_attr(fn, &per_sm);
  if (e != cudaSuccess) return e;
  const int grid = (int)std::min<int64_t>((int64_t)num_sms * per_sm, g.plan.nchunks);
  void *args[] = {(void *)&g};
  e = cudaLaunchKernel(fn, dim3(grid), dim3(kSThreads), args, sizeof(SplitSmem), st);
  if (e != cudaSuccess) return e;
  ++g_launches;
  return cudaGetLastError();
}

cudaError_t group_scatter2(const GroupArgs &g, cudaStream_t st) {
  const int64_t nq1 = (int64_t)g.plan.c * g.plan.nb1;
  if (nq1 == 0 || g.plan.bits == g.plan.bits1) return cudaSuccess;
  if (g.plan.bits - g.plan.bits1 > kMaxBits - kCoarseBits) return cudaErrorInvalidValue;
  const int fbits = (g.plan.bits1 == kCoarseBits &&
                     (g.plan.bits == 18 || g.plan.bits == 16 || g.plan.bits == 15))
                        ? g.plan.bits - kCoarseBits : 0;
  const int mode = split_mode(true);
  const void *fn = nullptr;
  switch (fbits * 4 + mode) {
#define SG_SC(F, M) case F * 4 + M: fn = (const void *)scatter2_kernel<F, M>; break;
    SG_SC(10, 0) SG_SC(10, 1) SG_SC(10, 2) SG_SC(10, 3)
    SG_SC(8, 0) SG_SC(8, 1) SG_SC(8, 2) SG_SC(8, 3)
    SG_SC(7, 0) SG_SC(7, 1) SG_SC(7, 2) SG_SC(7, 3)
    SG_SC(0, 0) SG_SC(0, 1) SG_SC(0, 2) SG_SC(0, 3)
#undef SG_SC
  }
  const size_t sm2 = (fbits == 0 || fbits > 8) ? sizeof(SplitSmemT<kMaxFine>) : sizeof(SplitSmem);
  int per_sm = 1;
  cudaError_t e = split_attr(fn, &per_sm, sm2);
  if (e != cudaSuccess) return e;
  void *args[] = {(void *)&g};
  e = cudaLaunchKernel(fn, dim3((unsigned)nq1), dim3(kSThreads), args, sm2, st);
  if (e != cudaSuccess) return e;
  ++g_launches;
  return cudaGetLastError();
}

cudaError_t popcount_words(const uint32_t *w, int64_t nwords, unsigned long long *d_out,
                           cudaStream_t st) {
  cudaError_t e = cudaMemsetAsync(d_out, 0, sizeof(unsigned long long), st);
  if (e != cudaSuccess) return e;
  if (nwords == 0) return cudaSuccess;
  int grid = (int)std::min<int64_t>((nwords + 255) / 256, 148 * 8);
  popcount_kernel<<<grid, 256, 0, st>>>(w, nwords, d_out);
  return cudaGetLastError();
}

cudaError_t sum_i32(const int32_t *a, int64_t n, unsigned long long *d_out, cudaStream_t st) {
  cudaError_t e = cudaMemsetAsync(d_out, 0, sizeof(unsigned long long), st);
  if (e != cudaSuccess || n == 0) return e;
  int grid = (int)std::min<int64_t>((n + 255) / 256, 148 * 8);
  sum_i32_kernel<<<grid, 256, 0, st>>>(a, n, d_out);
  return cudaGetLastError();
}

}  // namespace sg
