// kernels_sort.cu — per-trial grouping of <shingle, generator> pairs
// ("a sorting is done to gather all vertices that generated each shingle ...
// once for each random trial", AMB-5), second design
// (DESIGN.md §6.2): ONE stable partition pass by the top B <= 13 key bits,
// then one CTA per final bucket sorts it in shared memory.
//
//   1. hist    : per (trial, super-chunk of <= 64K pairs) histogram of the
//                B-bit bin (shared-memory counters, one read of the keys);
//   2. offsets : column prefix over the super-chunks of a trial + bucket
//                starts (kernels_group.cu colscan / binscan);
//   3. scatter : persistent 1024-thread CTAs.  A super-chunk is processed in
//                8K-pair sub-chunks: the keys are staged in shared memory,
//                ranked stably by bin with one or two LSD digit passes
//                (warp-private digit counters, __match_any_sync peers, the
//                rank of an element is fixed in the counting sweep so the
//                placement is one independent store per element), and the
//                pairs are written out in bin order: consecutive threads
//                write consecutive positions of a bucket (coalesced runs),
//                per-bin cursors carried across the super-chunk's
//                sub-chunks in shared memory (stable across sub-chunks);
//   4. local   : one 1024-thread CTA per bucket (<= 16K pairs, ~10K on the
//                2M graph's level II): keys staged in shared memory, two
//                8-bit LSD passes on the 16 key bits after the bin bits,
//                the rare runs of distinct keys sharing those 16 bits sorted
//                by insertion (stable), then members written in order with
//                one head bit per group start (ballot).  Larger buckets (a
//                group of many thousand generators) go to big_kernel
//                (kernels_local.cu), which sorts in global memory.
// Every step is stable and each trial's pairs enter in generator order, so
// the members of a group come out ascending: the canonical (key, member)
// order of the oracle (AMB-19).
#include <algorithm>
#include <cstdlib>

#include "group_common.cuh"
#include "kernels.h"
#include "scan.cuh"
#include "sg_internal.cuh"

namespace sg {

namespace {

using grp::bucket_extent;

constexpr int kXT = 1024;                 // threads of the scatter / local CTAs
constexpr int kXW = kXT / 32;
constexpr int kSub = 8192;                // pairs per scatter sub-chunk
constexpr int kXPer = kSub / kXT;         // 8 per thread
constexpr int kSuper = 65536;             // pairs per super-chunk (hist / cursor unit)
constexpr int kMaxB = 13;
constexpr int kMaxBins = 1 << kMaxB;
constexpr int kMaxDigitBits = 8;
constexpr int kLCap = 16384;              // local sort capacity (pairs per bucket)
constexpr int kLPer = kLCap / kXT;        // 16 per thread
constexpr int kMaxFix = 256;

__device__ __forceinline__ uint32_t lanemask_lt() {
  uint32_t m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}

__device__ __forceinline__ uint32_t bin_of(uint64_t key, int B) {
  return B ? (uint32_t)(key >> (64 - B)) : 0u;
}

// nbits (1..8) key bits starting `lo` bits below the MSB
__device__ __forceinline__ uint32_t digit_of(uint64_t key, int lo, int nbits) {
  return (uint32_t)((key << lo) >> (64 - nbits));
}

__device__ __forceinline__ uint32_t val_at2(const GroupArgs &g, int64_t in_idx, int64_t i) {
  if (g.vals) return g.vals[in_idx];
  if (g.rowid) return g.rowid[i];
  return g.val_base + (uint32_t)i;
}

// One stable LSD digit pass over the n <= 16384 elements of a CTA: the
// elements in order src (identity if null) are ranked by digit
// d = digit_of(K[e], lo, nbits) and their indices written to dst in (d, src
// position) order.  Warp w owns the contiguous positions [w*seg, (w+1)*seg);
// in its counting sweep each element gets its offset among the warp's
// earlier same-digit elements (a returning shared atomic on the warp's
// private counter by the lowest peer of its __match_any_sync group), so after
// one digit-major, warp-minor scan of the counters the placement is a single
// store per element.  cnt: (1 << nbits) * kXW packed u16 counters.
template <int PER>
__device__ __forceinline__ void rank_pass(const uint64_t *__restrict__ K, const uint16_t *src,
                                          uint16_t *dst, int n, int lo, int nbits, uint32_t *cnt,
                                          int64_t *ws) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const int nd = 1 << nbits;
  const int ncnt = nd * kXW;                       // u16 entries, digit-major
  uint16_t *c16 = reinterpret_cast<uint16_t *>(cnt);
  for (int i = threadIdx.x; i < (ncnt >> 1); i += kXT) cnt[i] = 0;
  const int seg = (((n + kXW - 1) / kXW) + 31) & ~31;   // positions per warp (<= PER * 32)
  const uint32_t lt = lanemask_lt();
  const int half = (w & 1) << 4;                   // warps w, w^1 share a counter word
  __syncthreads();
  uint32_t pk[PER];                                // e | offset << 14 | d << 24
#pragma unroll
  for (int u = 0; u < PER; ++u) {
    pk[u] = 0;
    if (u * 32 < seg) {                            // warp-uniform
      const int pos = w * seg + u * 32 + lane;
      const bool valid = pos < n;
      const uint32_t e = valid ? (src ? (uint32_t)src[pos] : (uint32_t)pos) : 0u;
      const uint32_t d = valid ? digit_of(K[e], lo, nbits) : 0xFFFFFFFFu;
      const uint32_t peers = __match_any_sync(0xffffffffu, d);
      const int leader = __ffs(peers) - 1;
      uint32_t old = 0;
      if (valid && lane == leader)
        old = atomicAdd(&cnt[(d * kXW + w) >> 1], (uint32_t)__popc(peers) << half);
      old = __shfl_sync(0xffffffffu, old, leader);
      const uint32_t off = ((old >> half) & 0xFFFFu) + (uint32_t)__popc(peers & lt);
      if (valid) pk[u] = e | (off << 14) | (d << 24);
    }
  }
  __syncthreads();
  {
    // exclusive scan of the counters in digit-major, warp-minor order
    const int per = (ncnt + kXT - 1) / kXT;        // 8 (8-bit digits) .. 1
    const int b0 = threadIdx.x * per;
    uint32_t s = 0;
    for (int x = 0; x < per; ++x)
      if (b0 + x < ncnt) s += c16[b0 + x];
    int64_t tot;
    uint32_t run = (uint32_t)block_excl_scan<int64_t>((int64_t)s, ws, &tot);
    for (int x = 0; x < per; ++x)
      if (b0 + x < ncnt) {
        const uint32_t v = c16[b0 + x];
        c16[b0 + x] = (uint16_t)run;
        run += v;
      }
  }
  __syncthreads();
#pragma unroll
  for (int u = 0; u < PER; ++u) {
    if (u * 32 < seg) {
      const int pos = w * seg + u * 32 + lane;
      if (pos < n) {
        const uint32_t v = pk[u];
        const uint32_t d = v >> 24;
        dst[c16[d * kXW + w] + ((v >> 14) & 0x3FFu)] = (uint16_t)(v & 0x3FFFu);
      }
    }
  }
  __syncthreads();
}

// ---- 1. histogram of the bin per super-chunk ---------------------------------
__global__ void __launch_bounds__(kXT) hist_b_kernel(const __grid_constant__ GroupArgs g) {
  extern __shared__ uint32_t hsm[];
  const int B = g.plan.bits;
  const int nb = 1 << B;
  for (int i = threadIdx.x; i < nb; i += kXT) hsm[i] = 0;
  __syncthreads();
  const int64_t k = blockIdx.x;
  const uint64_t *__restrict__ keys = g.keys + g.plan.chunk_in0[k];
  const int len = g.plan.chunk_len[k];
  int i = threadIdx.x;
  for (; i + 3 * kXT < len; i += 4 * kXT) {
    const uint64_t k0 = keys[i], k1 = keys[i + kXT], k2 = keys[i + 2 * kXT], k3 = keys[i + 3 * kXT];
    atomicAdd(&hsm[bin_of(k0, B)], 1u);
    atomicAdd(&hsm[bin_of(k1, B)], 1u);
    atomicAdd(&hsm[bin_of(k2, B)], 1u);
    atomicAdd(&hsm[bin_of(k3, B)], 1u);
  }
  for (; i < len; i += kXT) atomicAdd(&hsm[bin_of(keys[i], B)], 1u);
  __syncthreads();
  uint32_t *out = g.counts + k * nb;
  for (int b = threadIdx.x; b < nb; b += kXT) out[b] = hsm[b];
}

// ---- 3. stable partition by bin -----------------------------------------------
struct XSmem {
  uint64_t K[kSub];                 // staged keys of the sub-chunk
  uint16_t P0[kSub];                // order after the low digit pass
  uint16_t P1[kSub];                // order by bin
  uint16_t SB[kSub];                // bin of sorted position p
  uint32_t cur[kMaxBins];           // per-bin output cursor (trial-segment relative)
  uint32_t cnt[(1 << kMaxDigitBits) * kXW / 2];
  int64_t ws[33];
};

__global__ void __launch_bounds__(kXT, 1) scatter_b_kernel(const __grid_constant__ GroupArgs g) {
  extern __shared__ __align__(16) unsigned char smraw[];
  XSmem &S = *reinterpret_cast<XSmem *>(smraw);
  const int B = g.plan.bits;
  const int nb = 1 << B;
  const int bA = B > kMaxDigitBits ? (B + 1) / 2 : B;    // low (first) digit
  const int bB = B - bA;                                  // high digit (0: single pass)
  for (int64_t k = blockIdx.x; k < g.plan.nchunks; k += gridDim.x) {
    const int j = g.plan.chunk_trial[k];
    const int64_t in0 = g.plan.chunk_in0[k], i0 = g.plan.chunk_i0[k];
    const int L = g.plan.chunk_len[k];
    const int64_t sseg = g.plan.seg[j] - g.plan.seg[0];
    for (int b = threadIdx.x; b < nb; b += kXT)
      S.cur[b] = g.bstart1[(int64_t)j * nb + b] + g.counts[k * nb + b];
    for (int s0 = 0; s0 < L; s0 += kSub) {
      const int len = min(kSub, L - s0);
#pragma unroll
      for (int u = 0; u < kXPer; ++u) {
        const int i = threadIdx.x + u * kXT;
        if (i < len) S.K[i] = g.keys[in0 + s0 + i];
      }
      __syncthreads();
      const uint16_t *perm = nullptr;             // identity (one bin)
      if (B > 0) {
        if (bB == 0) {
          rank_pass<kXPer>(S.K, nullptr, S.P1, len, 0, B, S.cnt, S.ws);
        } else {
          rank_pass<kXPer>(S.K, nullptr, S.P0, len, B - bA, bA, S.cnt, S.ws);
          rank_pass<kXPer>(S.K, S.P0, S.P1, len, 0, bB, S.cnt, S.ws);
        }
        perm = S.P1;
      }
      // bins of the sorted positions; cursor -> offset at the start of each run
#pragma unroll
      for (int u = 0; u < kXPer; ++u) {
        const int p = threadIdx.x + u * kXT;
        if (p < len) S.SB[p] = (uint16_t)bin_of(S.K[perm ? perm[p] : p], B);
      }
      __syncthreads();
#pragma unroll
      for (int u = 0; u < kXPer; ++u) {
        const int p = threadIdx.x + u * kXT;
        if (p < len) {
          const uint32_t b = S.SB[p];
          if (p == 0 || S.SB[p - 1] != b) S.cur[b] -= (uint32_t)p;
        }
      }
      __syncthreads();
      // pairs out in bin order: consecutive positions of a run are consecutive
      // output positions of that bucket
#pragma unroll
      for (int u = 0; u < kXPer; ++u) {
        const int p = threadIdx.x + u * kXT;
        if (p < len) {
          const int e = perm ? perm[p] : p;
          const uint32_t o = S.cur[S.SB[p]] + (uint32_t)p;
          g.akeys[sseg + o] = S.K[e];
          g.avals[sseg + o] = val_at2(g, in0 + s0 + e, i0 + s0 + e);
        }
      }
      __syncthreads();
#pragma unroll
      for (int u = 0; u < kXPer; ++u) {
        const int p = threadIdx.x + u * kXT;
        if (p < len) {
          const uint32_t b = S.SB[p];
          if (p == len - 1 || S.SB[p + 1] != b) S.cur[b] += (uint32_t)p + 1u;
        }
      }
      __syncthreads();
    }
  }
}

// ---- 4. bucket sort + run-length segmentation ---------------------------------
struct LSmem {
  uint64_t K[kLCap];
  uint16_t P0[kLCap];
  uint16_t P1[kLCap];
  uint32_t cnt[(1 << kMaxDigitBits) * kXW / 2];
  uint32_t hb[kLCap / 32 + 2];
  uint32_t fix[kMaxFix];
  uint32_t nfix;
  int64_t ws[33];
};

// Merge bucket-local head words hb[0, nw) (bit p = position p) into the
// global head bit array at bit offset gbase; interior words are stored, the
// two boundary words (shared with neighbouring buckets) are OR-ed.
__device__ __forceinline__ void store_heads_b(uint32_t *head, const uint32_t *hb, int64_t gbase,
                                              int n) {
  const int64_t w0 = gbase >> 5, w1 = (gbase + n - 1) >> 5;
  const int off = (int)(gbase & 31);
  const int nw = (n + 31) >> 5;
  for (int64_t w = w0 + threadIdx.x; w <= w1; w += kXT) {
    const int k = (int)(w - w0);
    uint32_t bits;
    if (off == 0) {
      bits = k < nw ? hb[k] : 0u;
    } else {
      const uint32_t lo = (k >= 1 && k - 1 < nw) ? hb[k - 1] : 0u;
      const uint32_t hi = k < nw ? hb[k] : 0u;
      bits = (lo >> (32 - off)) | (hi << off);
    }
    const int64_t lo_pos = w << 5, hi_pos = lo_pos + 32;
    if (lo_pos >= gbase && hi_pos <= gbase + n) head[w] = bits;
    else if (bits) atomicOr(&head[w], bits);
  }
}

__global__ void __launch_bounds__(kXT, 1) local_b_kernel(const __grid_constant__ GroupArgs g) {
  extern __shared__ __align__(16) unsigned char smraw[];
  LSmem &S = *reinterpret_cast<LSmem *>(smraw);
  const int B = g.plan.bits;
  const int64_t nq = (int64_t)g.plan.c * g.plan.nbins;
  const int64_t obase = g.plan.seg[0];
  const int cap = g.plan.local_cap;
  const int lo2 = B, lo1 = B + 8;                 // LSD: bits [B+8, B+16) first, then [B, B+8)
  for (int64_t q = blockIdx.x; q < nq; q += gridDim.x) {
    int64_t sb, n64;
    bucket_extent(g, q, sb, n64);
    if (n64 == 0) continue;
    if (n64 > cap) {
      if (threadIdx.x == 0) g.big_list[atomicAdd(g.big_count, 1u)] = (uint32_t)q;
      continue;
    }
    const int n = (int)n64;
    const uint64_t *__restrict__ Kg = g.bkeys + sb;
    const uint32_t *__restrict__ Vg = g.bvals + sb;
#pragma unroll
    for (int u = 0; u < kLPer; ++u) {
      const int i = threadIdx.x + u * kXT;
      if (i < n) S.K[i] = Kg[i];
    }
    __syncthreads();
    const uint16_t *pm;
    if (n > 1) {
      rank_pass<kLPer>(S.K, nullptr, S.P0, n, lo1, 8, S.cnt, S.ws);
      rank_pass<kLPer>(S.K, S.P0, S.P1, n, lo2, 8, S.cnt, S.ws);
      // distinct keys sharing the 16 sorted bits out of key order: mark the
      // start of each such run, sort each run by key (stable insertion)
      for (int i = threadIdx.x; i < (kLCap / 32 + 2); i += kXT) S.hb[i] = 0;
      if (threadIdx.x == 0) S.nfix = 0;
      __syncthreads();
      for (int p = threadIdx.x + 1; p < n; p += kXT) {
        const uint64_t kp = S.K[S.P1[p]];
        if (kp < S.K[S.P1[p - 1]]) {
          const uint32_t dp = digit_of(kp, lo2, 16);
          int a = p - 1;
          while (a > 0 && digit_of(S.K[S.P1[a - 1]], lo2, 16) == dp) --a;
          const uint32_t bit = 1u << (a & 31);
          if (!(atomicOr(&S.hb[a >> 5], bit) & bit)) {
            const uint32_t s = atomicAdd(&S.nfix, 1u);
            if (s < kMaxFix) S.fix[s] = (uint32_t)a;
          }
        }
      }
      __syncthreads();
      const uint32_t nfix = S.nfix;
      uint16_t *q2 = S.P1;
      if (nfix > kMaxFix) {
        // pathological: one stable insertion sort of the whole bucket
        if (threadIdx.x == 0) {
          for (int x = 1; x < n; ++x) {
            const uint16_t e = q2[x];
            const uint64_t ke = S.K[e];
            int y = x - 1;
            while (y >= 0 && ke < S.K[q2[y]]) { q2[y + 1] = q2[y]; --y; }
            q2[y + 1] = e;
          }
        }
      } else if (threadIdx.x < (int)nfix) {
        const int a = (int)S.fix[threadIdx.x];
        const uint32_t da = digit_of(S.K[q2[a]], lo2, 16);
        int b = a + 1;
        while (b < n && digit_of(S.K[q2[b]], lo2, 16) == da) ++b;
        for (int x = a + 1; x < b; ++x) {
          const uint16_t e = q2[x];
          const uint64_t ke = S.K[e];
          int y = x - 1;
          while (y >= a && ke < S.K[q2[y]]) { q2[y + 1] = q2[y]; --y; }   // strict: stable
          q2[y + 1] = e;
        }
      }
      __syncthreads();
      pm = S.P1;
    } else {
      S.P1[0] = 0;
      __syncthreads();
      pm = S.P1;
    }
    // members in sorted order, one head bit per group start (ballot per warp row)
    const int64_t gbase = obase + sb;
    const int lane = threadIdx.x & 31;
#pragma unroll
    for (int u = 0; u < kLPer; ++u) {
      const int p = threadIdx.x + u * kXT;
      if (u * kXT < n) {                                  // block-uniform
        bool head = false;
        if (p < n) {
          const int e = pm[p];
          const uint64_t key = S.K[e];
          g.members[gbase + p] = Vg[e];
          if (g.okeys) g.okeys[gbase + p] = key;
          head = (p == 0) || S.K[pm[p - 1]] != key;
        }
        const uint32_t hw = __ballot_sync(0xffffffffu, head);
        if (lane == 0) S.hb[p >> 5] = hw;
      }
    }
    __syncthreads();
    store_heads_b(g.head, S.hb, gbase, n);
    __syncthreads();
  }
}

}  // namespace

int64_t group_b_super_pairs() { return kSuper; }
int32_t group_b_max_bits() { return kMaxB; }
int32_t group_b_local_cap() { return kLCap; }

void group_b_bits(int64_t maxseg, int32_t *bits) {
  // buckets of ~10K pairs on average (the local sort holds 16K)
  // test hook SG_GROUP_TARGET: smaller average buckets (more bins)
  const char *e = getenv("SG_GROUP_TARGET");
  int64_t target = e ? atoll(e) : 10240;
  if (target <= 0) target = 10240;
  int b = 0;
  while ((maxseg >> b) > target && b < kMaxB) ++b;
  *bits = b;
}

cudaError_t group_b_hist(const GroupArgs &a, cudaStream_t st) {
  if (a.plan.nchunks == 0) return cudaSuccess;
  const int B = a.plan.bits;
  if (B < 0 || B > kMaxB) return cudaErrorInvalidValue;
  const int nb = 1 << B;
  hist_b_kernel<<<(unsigned)a.plan.nchunks, kXT, (size_t)nb * 4, st>>>(a);
  ++g_launches;
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return e;
  GroupArgs o = a;
  o.plan.nb1 = nb;
  return group_offsets(o, st);
}

cudaError_t group_b_scatter(const GroupArgs &a, int num_sms, cudaStream_t st) {
  if (a.plan.nchunks == 0) return cudaSuccess;
  if (a.plan.bits < 0 || a.plan.bits > kMaxB) return cudaErrorInvalidValue;
  const size_t smem = sizeof(XSmem);
  cudaError_t e = cudaFuncSetAttribute(scatter_b_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       (int)smem);
  if (e != cudaSuccess) return e;
  const int grid = (int)std::min<int64_t>(num_sms, a.plan.nchunks);
  scatter_b_kernel<<<grid, kXT, smem, st>>>(a);
  ++g_launches;
  return cudaGetLastError();
}

cudaError_t group_b_local(const GroupArgs &a0, int num_sms, cudaStream_t st) {
  GroupArgs a = a0;
  if (a.plan.local_cap <= 0 || a.plan.local_cap > kLCap) a.plan.local_cap = kLCap;
  const int64_t nq = (int64_t)a.plan.c * a.plan.nbins;
  if (nq == 0) return cudaSuccess;
  const size_t smem = sizeof(LSmem);
  cudaError_t e = cudaFuncSetAttribute(local_b_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       (int)smem);
  if (e != cudaSuccess) return e;
  const int grid = (int)std::min<int64_t>(num_sms, nq);
  local_b_kernel<<<grid, kXT, smem, st>>>(a);
  ++g_launches;
  if ((e = cudaGetLastError()) != cudaSuccess) return e;
  return group_big(a, num_sms, st);     // oversize buckets (list length read on the device)
}

}  // namespace sg
