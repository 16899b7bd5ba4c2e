// kernels_local.cu — sort inside one key bucket and run-length segmentation:
// the second half of the per-trial grouping (AMB-5).
//
// The partition (kernels_group.cu) is stable in practice, so inside a bucket
// the pairs of one trial are in generator order and a stable sort by key
// alone yields the canonical (key, member) order.  The warp tier (default)
// and the CTA tier verify the full (key, member) order while writing and
// re-sort every violating run by (key, member), so the result is canonical
// whatever order the partition delivered.
//
// Three tiers by bucket size n (mean ~600 pairs):
//  * warp_local_kernel (n <= 1024): one warp per bucket, no block barriers.
//    One sweep over the bucket's keys stores the 20 key bits after the
//    bucket bits in the warp's shared-memory slice and builds both 10-bit
//    digit histograms (packed 16-bit shared atomics); two LSD placement
//    passes sort an index permutation, each element taking its slot with its
//    own returning shared atomic (no __match_any_sync; SG_LOCAL_ATOMIC=0
//    selects the match-based stable placement); members are gathered through
//    L1 and written in order (coalesced) with one head bit per group start.
//    The rare equal-high-digit runs found out of (key, member) order while
//    writing (20-bit ties, or lanes served out of order) are re-sorted by
//    (key, member) and written again.  Larger buckets are appended to the
//    mid / big lists.
//  * local_kernel (n <= 4096, mid list): the same passes by a 256-thread CTA.
//  * big_kernel (n > 4096, big list; groups of huge cliques): one CTA per
//    bucket, bitonic sort by (key, member) in global (L2-resident) memory.
// The mid and big tiers read their list lengths on the device (no host sync).
#include <algorithm>
#include <cstdlib>

#include "group_common.cuh"
#include "kernels.h"
#include "scan.cuh"
#include "sg_internal.cuh"

namespace sg {

namespace {

using grp::bucket_extent;
using grp::pair_less;

__device__ __forceinline__ uint32_t lanemask_lt() {
  uint32_t m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}

__device__ __forceinline__ void cp_async(void *sdst, const void *gsrc, int bytes) {
  const unsigned s = (unsigned)__cvta_generic_to_shared(sdst);
  if (bytes == 8) asm volatile("cp.async.ca.shared.global [%0], [%1], 8;\n" ::"r"(s), "l"(gsrc));
  else asm volatile("cp.async.ca.shared.global [%0], [%1], 4;\n" ::"r"(s), "l"(gsrc));
}

__device__ __forceinline__ void cp_async_wait_all() {
  asm volatile("cp.async.commit_group;\ncp.async.wait_all;\n" ::);
}

// Merge bucket-local head words hb[0, nw) (bit p = position p) into the
// global head bit array at bit offset gbase; interior words are stored,
// the two boundary words (shared with neighbouring buckets) are OR-ed.
__device__ __forceinline__ void store_heads(uint32_t *head, const uint32_t *hb, int64_t gbase,
                                            int n, int tid, int nthr) {
  const int64_t w0 = gbase >> 5, w1 = (gbase + n - 1) >> 5;
  const int off = (int)(gbase & 31);
  const int nw = (n + 31) >> 5;
  for (int64_t w = w0 + tid; w <= w1; w += nthr) {
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

constexpr int kLocalCap = 4096;            // CTA tier capacity

// ============================================================ warp tier
constexpr int kWCap = 1024;
constexpr int kWBatch = kWCap / 32;        // 32 batches of 32 positions
constexpr int kWWarps = 7;                 // warps per CTA (3 CTAs, 21 warps per SM)
constexpr int kWDigitBits = 10;            // two LSD passes = 20 key bits
constexpr int kWDigits = 1 << kWDigitBits;
constexpr int kWB = 8;                     // batches of 32 in flight (placement, emit)

struct __align__(16) WarpSmem {
  uint32_t d20[kWCap];        // the 20 key bits after the bucket bits
  uint16_t pa[kWCap];         // order after the first pass
  uint16_t cA[kWDigits];      // low-digit counts -> cursors; then the final order
  uint16_t cB[kWDigits];      // high-digit counts -> cursors
  uint32_t hb[kWBatch];
};

// Exclusive scan in place of 1024 uint16 counters (lane owns 32 consecutive).
__device__ __forceinline__ void warp_scan_1024(uint16_t *cnt) {
  const int lane = threadIdx.x & 31;
  uint32_t *w32 = reinterpret_cast<uint32_t *>(cnt) + lane * 16;
  uint32_t v[16];
  uint32_t s = 0;
#pragma unroll
  for (int x = 0; x < 16; ++x) {
    v[x] = w32[x];
    s += (v[x] & 0xFFFFu) + (v[x] >> 16);
  }
  uint32_t run = warp_incl_scan(s) - s;
#pragma unroll
  for (int x = 0; x < 16; ++x) {
    const uint32_t lo = run;
    const uint32_t hi = run + (v[x] & 0xFFFFu);
    run = hi + (v[x] >> 16);
    w32[x] = lo | (hi << 16);
  }
}

// Stable placement pass: position of element e (visited in the order src,
// identity if FIRST) = cursor[digit] + rank among same-digit peers of its
// batch (__match_any_sync, converged with the full mask; invalid lanes carry
// the sentinel digit kWDigits); the lowest peer advances the packed-u16
// cursor with a returning shared atomic, four batches in flight.
// ATOMIC: every element takes its slot with its own returning shared atomic
// (no __match_any_sync: its latency headed the kernel's stall list).  The
// order of same-address atomics within one warp instruction is not
// specified, so the placement may be unstable; warp_emit then verifies the
// full (key, member) order and the caller re-sorts the violating runs.
template <bool FIRST, bool ATOMIC>
__device__ __forceinline__ void warp_place(const WarpSmem &S, int n, const uint16_t *src,
                                           uint16_t *cur, uint16_t *dst, int shift) {
  const int lane = threadIdx.x & 31;
  const uint32_t lt = lanemask_lt();
  uint32_t *cw = reinterpret_cast<uint32_t *>(cur);
  if (ATOMIC) {
    for (int i0 = 0; i0 < n; i0 += 32 * kWB) {
      uint32_t e[kWB], d[kWB], o[kWB];
#pragma unroll
      for (int u = 0; u < kWB; ++u) {
        const int i = i0 + u * 32 + lane;
        const bool valid = i < n;
        e[u] = valid ? (FIRST ? (uint32_t)i : (uint32_t)src[i]) : 0u;
        d[u] = valid ? (S.d20[e[u]] >> shift) & (kWDigits - 1) : 0u;
        o[u] = valid ? atomicAdd(&cw[d[u] >> 1], 1u << ((d[u] & 1) << 4)) : 0u;
      }
#pragma unroll
      for (int u = 0; u < kWB; ++u)
        if (i0 + u * 32 + lane < n) dst[(o[u] >> ((d[u] & 1) << 4)) & 0xFFFFu] = (uint16_t)e[u];
    }
    __syncwarp();
    return;
  }
  for (int i0 = 0; i0 < n; i0 += 32 * kWB) {
    uint32_t e[kWB], d[kWB], m[kWB], o[kWB];
#pragma unroll
    for (int u = 0; u < kWB; ++u) {
      const int i = i0 + u * 32 + lane;
      const bool valid = i < n;
      e[u] = valid ? (FIRST ? (uint32_t)i : (uint32_t)src[i]) : 0u;
      d[u] = valid ? (S.d20[e[u]] >> shift) & (kWDigits - 1) : (uint32_t)kWDigits;
      m[u] = __match_any_sync(0xffffffffu, d[u]);   // (ballot-built masks measured slower here)
      o[u] = 0;
      if (valid && (m[u] & lt) == 0)
        o[u] = atomicAdd(&cw[d[u] >> 1], (uint32_t)__popc(m[u]) << ((d[u] & 1) << 4));
    }
#pragma unroll
    for (int u = 0; u < kWB; ++u) {
      const uint32_t oo = __shfl_sync(0xffffffffu, o[u], __ffs(m[u]) - 1);
      if (i0 + u * 32 + lane < n) {
        const uint32_t base = (oo >> ((d[u] & 1) << 4)) & 0xFFFFu;
        dst[base + __popc(m[u] & lt)] = (uint16_t)e[u];
      }
    }
  }
  __syncwarp();
}

// Write members (and sorted keys) in the order pm; head bits into S.hb.
// Returns true if some adjacent pair is out of key order (a 20-bit tie), or,
// with FULL, out of (key, member) order.
// Gathers of four batches are issued before their stores.
template <bool FULL>
__device__ __forceinline__ bool warp_emit(const GroupArgs &g, WarpSmem &S, int n,
                                          const uint16_t *pm, const uint64_t *__restrict__ Kg,
                                          const uint32_t *__restrict__ Vg, int64_t gbase) {
  const int lane = threadIdx.x & 31;
  bool bad = false;
  uint64_t carry = 0;
  uint32_t carryv = 0;
  for (int p0 = 0; p0 < n; p0 += 32 * kWB) {
    int e[kWB];
    uint64_t ke[kWB];
    uint32_t ve[kWB];
#pragma unroll
    for (int u = 0; u < kWB; ++u) {
      const int p = p0 + u * 32 + lane;
      e[u] = p < n ? pm[p] : 0;
    }
#pragma unroll
    for (int u = 0; u < kWB; ++u) {
      const bool valid = p0 + u * 32 + lane < n;
      ke[u] = valid ? Kg[e[u]] : ~0ull;
      ve[u] = valid ? Vg[e[u]] : 0u;
    }
#pragma unroll
    for (int u = 0; u < kWB; ++u) {
      if (p0 + u * 32 >= n) break;                    // warp-uniform
      const int p = p0 + u * 32 + lane;
      const bool valid = p < n;
      uint64_t prev = __shfl_up_sync(0xffffffffu, ke[u], 1);
      if (lane == 0) prev = carry;
      carry = __shfl_sync(0xffffffffu, ke[u], 31);
      uint32_t prevv = 0;
      if (FULL) {
        prevv = __shfl_up_sync(0xffffffffu, ve[u], 1);
        if (lane == 0) prevv = carryv;
        carryv = __shfl_sync(0xffffffffu, ve[u], 31);
      }
      bool head = false;
      if (valid) {
        g.members[gbase + p] = ve[u];
        if (g.okeys) g.okeys[gbase + p] = ke[u];
        head = (p == 0) || prev != ke[u];
        bad |= (p > 0) && (ke[u] < prev || (FULL && ke[u] == prev && ve[u] < prevv));
      }
      const uint32_t hw = __ballot_sync(0xffffffffu, head);
      if (lane == 0) S.hb[(p0 >> 5) + u] = hw;
    }
  }
  return __any_sync(0xffffffffu, bad);
}

// BITS > 0: the plan's bucket bits known at compile time (16: the level-II
// plans of the 2M / 640M configs), so the sort digits are constant shifts.
// ATOMIC: atomic (possibly unstable) placements + full-order verification.
template <int BITS, bool ATOMIC>
__global__ void __launch_bounds__(kWWarps * 32, 3) warp_local_kernel(const __grid_constant__ GroupArgs g) {
  extern __shared__ __align__(16) unsigned char smraw[];
  const int lane = threadIdx.x & 31, wl = threadIdx.x >> 5;
  WarpSmem &S = reinterpret_cast<WarpSmem *>(smraw)[wl];
  const int64_t nq = (int64_t)g.plan.c * g.plan.nbins;
  const int bits = BITS > 0 ? BITS : g.plan.bits;
  const int64_t obase = g.plan.seg[0];     // scratch -> output position
  const int64_t nwarps = (int64_t)gridDim.x * kWWarps;
  for (int64_t q = (int64_t)blockIdx.x * kWWarps + wl; q < nq; q += nwarps) {
    int64_t sb, n64;
    bucket_extent(g, q, sb, n64);
    if (n64 == 0) continue;
    if (n64 > kWCap) {
      if (lane == 0) {
        if (n64 > kLocalCap) g.big_list[atomicAdd(g.big_count, 1u)] = (uint32_t)q;
        else g.mid_list[atomicAdd(g.mid_count, 1u)] = (uint32_t)q;
      }
      continue;
    }
    const int n = (int)n64;
    const uint64_t *Kg = g.bkeys + sb;
    const uint32_t *Vg = g.bvals + sb;
    {
      uint4 *a4 = reinterpret_cast<uint4 *>(S.cA);
      uint4 *b4 = reinterpret_cast<uint4 *>(S.cB);
#pragma unroll
      for (int x = 0; x < kWDigits / 256; ++x) {
        a4[lane + 32 * x] = make_uint4(0, 0, 0, 0);
        b4[lane + 32 * x] = make_uint4(0, 0, 0, 0);
      }
    }
    __syncwarp();
    // one sweep: the 20 sort bits of each key and both digit histograms
    // (packed 16-bit counters, order-free); the values are prefetched into L1
    // eight key loads in flight per lane (ncu: the sweep's first use of a
    // key headed the kernel's stall list with four)
    for (int i0 = 0; i0 < n; i0 += 256) {
      uint64_t k4[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const int i = i0 + u * 32 + lane;
        k4[u] = i < n ? Kg[i] : 0ull;
      }
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const int i = i0 + u * 32 + lane;
        if (i < n) {
          const uint32_t d20 = (uint32_t)((k4[u] << bits) >> 44);
          S.d20[i] = d20;
          const uint32_t dl = d20 & (kWDigits - 1), dh = d20 >> kWDigitBits;
          atomicAdd(reinterpret_cast<uint32_t *>(S.cA) + (dl >> 1), 1u << (16 * (dl & 1)));
          atomicAdd(reinterpret_cast<uint32_t *>(S.cB) + (dh >> 1), 1u << (16 * (dh & 1)));
          asm volatile("prefetch.global.L1 [%0];" ::"l"(Vg + i));
        }
      }
    }
    __syncwarp();
    warp_scan_1024(S.cA);
    warp_scan_1024(S.cB);
    __syncwarp();
    warp_place<true, ATOMIC>(S, n, nullptr, S.cA, S.pa, 0);
    uint16_t *pm = S.cA;                    // the low-digit cursors are spent
    warp_place<false, ATOMIC>(S, n, S.pa, S.cB, pm, kWDigitBits);
    const int64_t gbase = obase + sb;
    if (ATOMIC && warp_emit<true>(g, S, n, pm, Kg, Vg, gbase)) {
      // some equal-high-digit run is out of (key, member) order (an unstable
      // atomic placement, or a 20-bit tie): re-sort each such run by (key,
      // member) — a strict total order, so the result is canonical — and
      // emit again
      __syncwarp();
      S.hb[lane] = 0;
      __syncwarp();
      for (int p = lane + 1; p < n; p += 32) {
        const uint16_t ep = pm[p], eq = pm[p - 1];
        if (pair_less(Kg[ep], Vg[ep], Kg[eq], Vg[eq])) {
          const uint32_t dp = S.d20[ep] >> kWDigitBits;
          int a = p - 1;
          while (a > 0 && (S.d20[pm[a - 1]] >> kWDigitBits) == dp) --a;
          atomicOr(&S.hb[a >> 5], 1u << (a & 31));
        }
      }
      __syncwarp();
      uint32_t word = S.hb[lane];
      __syncwarp();
      while (word) {
        const int a = lane * 32 + __ffs(word) - 1;
        word &= word - 1;
        const uint32_t da = S.d20[pm[a]] >> kWDigitBits;
        int b = a + 1;
        while (b < n && (S.d20[pm[b]] >> kWDigitBits) == da) ++b;
        for (int x = a + 1; x < b; ++x) {
          const uint16_t e = pm[x];
          const uint64_t ke = Kg[e];
          const uint32_t ve = Vg[e];
          int y = x - 1;
          while (y >= a && pair_less(ke, ve, Kg[pm[y]], Vg[pm[y]])) { pm[y + 1] = pm[y]; --y; }
          pm[y + 1] = e;
        }
      }
      __syncwarp();
      warp_emit<true>(g, S, n, pm, Kg, Vg, gbase);
    } else if (!ATOMIC && warp_emit<false>(g, S, n, pm, Kg, Vg, gbase)) {
      // distinct keys sharing the 20 bits out of key order: mark the start of
      // each such equal-20-bit run, sort each run by key (stable), emit again
      __syncwarp();
      S.hb[lane] = 0;
      __syncwarp();
      for (int p = lane + 1; p < n; p += 32) {
        const uint64_t kp = Kg[pm[p]];
        if (kp < Kg[pm[p - 1]]) {
          const uint32_t dp = S.d20[pm[p]];
          int a = p - 1;
          while (a > 0 && S.d20[pm[a - 1]] == dp) --a;
          atomicOr(&S.hb[a >> 5], 1u << (a & 31));
        }
      }
      __syncwarp();
      uint32_t word = S.hb[lane];
      __syncwarp();
      while (word) {
        const int a = lane * 32 + __ffs(word) - 1;
        word &= word - 1;
        const uint32_t da = S.d20[pm[a]];
        int b = a + 1;
        while (b < n && S.d20[pm[b]] == da) ++b;
        for (int x = a + 1; x < b; ++x) {
          const uint16_t e = pm[x];
          const uint64_t ke = Kg[e];
          int y = x - 1;
          while (y >= a && ke < Kg[pm[y]]) { pm[y + 1] = pm[y]; --y; }   // strict: stable
          pm[y + 1] = e;
        }
      }
      __syncwarp();
      warp_emit<false>(g, S, n, pm, Kg, Vg, gbase);
    }
    __syncwarp();
    store_heads(g.head, S.hb, gbase, n, lane, 32);
    __syncwarp();
  }
}

// ============================================================ CTA tier
constexpr int kLThreads = 256;
constexpr int kLWarps = kLThreads / 32;
constexpr int kPerLane = kLocalCap / kLThreads;   // 16
constexpr int kDigits = 256;
constexpr int kCntPerThread = kDigits * kLWarps / kLThreads;   // 8

struct LocalSmem {
  uint64_t K[kLocalCap];
  uint32_t V[kLocalCap];
  uint16_t perm[2][kLocalCap];
  uint16_t cnt[kDigits * kLWarps];   // bin-major: [digit][warp]
  uint32_t peers[kLocalCap];         // match masks (warp segments)
  uint32_t nfix;
  uint32_t fix[64];
  uint32_t hb[kLocalCap / 32 + 2];
  int64_t ws[33];
};
static_assert(kCntPerThread == 8, "counter scan assumes 8 per thread");

// One stable multi-split pass over n <= 4096 elements: warp w owns the
// positions [w*seg, (w+1)*seg) of the current order src (identity if null)
// and writes the new order to dst, stable on digit(key).  ATOMIC: every
// element counts and takes its slot with its own shared atomic on the
// (digit, warp) counter instead of __match_any_sync peers (stable when the
// hardware serves one instruction's conflicting lanes in lane order, as
// measured; the caller's (key, member) verification repairs it otherwise).
template <bool ATOMIC, typename DIG>
__device__ __forceinline__ void lsd_pass(LocalSmem &S, int n, const uint16_t *src, uint16_t *dst,
                                         DIG digit) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const uint32_t lt = lanemask_lt();
  const int seg = (n + kLWarps - 1) / kLWarps;     // <= 512
  reinterpret_cast<uint4 *>(S.cnt)[threadIdx.x] = make_uint4(0, 0, 0, 0);
  __syncthreads();
  if (ATOMIC) {
    uint32_t *cw = reinterpret_cast<uint32_t *>(S.cnt);
    const int seg_lo = w * seg, seg_hi = min(n, seg_lo + seg);
    for (int pos = seg_lo + lane; pos < seg_hi; pos += 32) {
      const int idx = (int)digit(S.K[src ? src[pos] : pos]) * kLWarps + w;
      atomicAdd(cw + (idx >> 1), 1u << ((idx & 1) << 4));
    }
    __syncthreads();
    {
      uint4 *c4 = reinterpret_cast<uint4 *>(S.cnt);
      uint4 v = c4[threadIdx.x];
      uint16_t *c = reinterpret_cast<uint16_t *>(&v);
      uint32_t s = 0, run[kCntPerThread];
#pragma unroll
      for (int x = 0; x < kCntPerThread; ++x) {
        run[x] = s;
        s += c[x];
      }
      int64_t tot;
      const int64_t ex = block_excl_scan<int64_t>((int64_t)s, S.ws, &tot);
#pragma unroll
      for (int x = 0; x < kCntPerThread; ++x) c[x] = (uint16_t)(ex + run[x]);
      c4[threadIdx.x] = v;
    }
    __syncthreads();
    for (int pos0 = seg_lo; pos0 < seg_hi; pos0 += 4 * 32) {
      uint32_t el[4], o[4];
      int id[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const int pos = pos0 + u * 32 + lane;
        el[u] = 0;
        o[u] = 0;
        id[u] = 0;
        if (pos < seg_hi) {
          el[u] = src ? src[pos] : (uint32_t)pos;
          id[u] = (int)digit(S.K[el[u]]) * kLWarps + w;
          o[u] = atomicAdd(cw + (id[u] >> 1), 1u << ((id[u] & 1) << 4));
        }
      }
#pragma unroll
      for (int u = 0; u < 4; ++u)
        if (pos0 + u * 32 + lane < seg_hi) dst[(o[u] >> ((id[u] & 1) << 4)) & 0xFFFFu] = (uint16_t)el[u];
    }
    __syncthreads();
    return;
  }
  uint32_t *pr = S.peers + w * kPerLane * 32;     // match masks of this warp
  const int seg_lo = w * seg, seg_hi = min(n, seg_lo + seg);
  for (int pos = seg_lo + lane; pos - lane < seg_hi; pos += 32) {   // warp-uniform trip count
    const bool valid = pos < seg_hi;
    const uint32_t vm = __ballot_sync(0xffffffffu, valid);
    if (valid) {
      const uint32_t dg = digit(S.K[src ? src[pos] : pos]);
      const uint32_t m = __match_any_sync(vm, dg);
      pr[pos - seg_lo] = m;
      if ((m & lt) == 0) S.cnt[dg * kLWarps + w] += (uint16_t)__popc(m);
    }
    __syncwarp();
  }
  __syncthreads();
  {
    // exclusive scan of the bin-major counters (8 per thread)
    uint4 *c4 = reinterpret_cast<uint4 *>(S.cnt);
    uint4 v = c4[threadIdx.x];
    uint16_t *c = reinterpret_cast<uint16_t *>(&v);
    uint32_t s = 0, run[kCntPerThread];
#pragma unroll
    for (int x = 0; x < kCntPerThread; ++x) {
      run[x] = s;
      s += c[x];
    }
    int64_t tot;
    const int64_t ex = block_excl_scan<int64_t>((int64_t)s, S.ws, &tot);
#pragma unroll
    for (int x = 0; x < kCntPerThread; ++x) c[x] = (uint16_t)(ex + run[x]);
    c4[threadIdx.x] = v;
  }
  __syncthreads();
  for (int pos = seg_lo + lane; pos - lane < seg_hi; pos += 32) {
    const bool valid = pos < seg_hi;
    const uint32_t vm = __ballot_sync(0xffffffffu, valid);
    if (valid) {
      const uint16_t el = src ? src[pos] : (uint16_t)pos;
      const uint32_t dg = digit(S.K[el]);
      const uint32_t m = pr[pos - seg_lo];
      const uint32_t rank = __popc(m & lt);
      const uint32_t base = S.cnt[dg * kLWarps + w];
      __syncwarp(vm);
      if (rank == 0) S.cnt[dg * kLWarps + w] = (uint16_t)(base + __popc(m));
      __syncwarp(vm);
      dst[base + rank] = el;
    }
    __syncwarp();
  }
  __syncthreads();
}

template <bool ATOMIC>
__global__ void __launch_bounds__(kLThreads, 2) local_kernel(const __grid_constant__ GroupArgs g) {
  extern __shared__ __align__(16) unsigned char smraw[];
  LocalSmem &S = *reinterpret_cast<LocalSmem *>(smraw);
  const int bits = g.plan.bits;
  const int64_t obase = g.plan.seg[0];     // scratch -> output position
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const uint32_t nmid = *g.mid_count;
  for (uint32_t li = blockIdx.x; li < nmid; li += gridDim.x) {
    const int64_t q = g.mid_list[li];
    int64_t sb, n64;
    bucket_extent(g, q, sb, n64);
    const int n = (int)n64;
    for (int i = threadIdx.x; i < n; i += kLThreads) {
      cp_async(&S.K[i], g.bkeys + sb + i, 8);
      cp_async(&S.V[i], g.bvals + sb + i, 4);
    }
    cp_async_wait_all();
    // (lsd_pass begins with a barrier after zeroing its counters)
    lsd_pass<ATOMIC>(S, n, nullptr, S.perm[0],
                     [&](uint64_t key) { return (uint32_t)((key << (bits + 8)) >> 56); });
    lsd_pass<ATOMIC>(S, n, S.perm[0], S.perm[1],
                     [&](uint64_t key) { return (uint32_t)((key << bits) >> 56); });
    const uint16_t *pm = S.perm[1];
    const uint64_t *K = S.K;
    // repair runs: equal 16 sorted bits, or (ATOMIC: the last pass may be
    // unstable only inside one high digit) equal high digit
    auto d16 = [&](uint64_t key) { return (uint32_t)((key << bits) >> (ATOMIC ? 56 : 48)); };
    // ---- rare: distinct keys sharing the 16 bits out of key order -> a
    // stable insertion sort of that run (registered once via its start bit)
    for (int i = threadIdx.x; i < (kLocalCap / 32 + 2); i += blockDim.x) S.hb[i] = 0;
    if (threadIdx.x == 0) S.nfix = 0;
    __syncthreads();
    // (the check and the repair use the full (key, member) order, so an
    // input that is not in generator order — atomic split ranking — is
    // repaired too)
    for (int p = threadIdx.x + 1; p < n; p += blockDim.x) {
      const uint64_t kp = K[pm[p]];
      if (pair_less(kp, S.V[pm[p]], K[pm[p - 1]], S.V[pm[p - 1]])) {
        const uint32_t dp = d16(kp);
        int a = p - 1;
        while (a > 0 && d16(K[pm[a - 1]]) == dp) --a;
        const uint32_t bit = 1u << (a & 31);
        if (!(atomicOr(&S.hb[a >> 5], bit) & bit)) {
          const uint32_t s = atomicAdd(&S.nfix, 1u);
          if (s < 64) S.fix[s] = (uint32_t)a;
        }
      }
    }
    __syncthreads();
    const uint32_t nfix = S.nfix;
    if (nfix > 64) {
      // pathological: one stable insertion sort of everything
      if (threadIdx.x == 0) {
        uint16_t *q2 = S.perm[1];
        for (int x = 1; x < n; ++x) {
          const uint16_t e = q2[x];
          const uint64_t ke = K[e];
          const uint32_t ve = S.V[e];
          int y = x - 1;
          while (y >= 0 && pair_less(ke, ve, K[q2[y]], S.V[q2[y]])) { q2[y + 1] = q2[y]; --y; }
          q2[y + 1] = e;
        }
      }
    } else if (threadIdx.x < (int)nfix) {
      uint16_t *q2 = S.perm[1];
      const int a = (int)S.fix[threadIdx.x];
      const uint32_t da = d16(K[q2[a]]);
      int b = a + 1;
      while (b < n && d16(K[q2[b]]) == da) ++b;
      for (int x = a + 1; x < b; ++x) {
        const uint16_t e = q2[x];
        const uint64_t ke = K[e];
        const uint32_t ve = S.V[e];
        int y = x - 1;
        while (y >= a && pair_less(ke, ve, K[q2[y]], S.V[q2[y]])) { q2[y + 1] = q2[y]; --y; }
        q2[y + 1] = e;
      }
    }
    __syncthreads();
    // ---- members in sorted order + head bits (ballot per 32 positions)
    const int64_t gbase = obase + sb;
    for (int p0 = w * 32; p0 < n; p0 += blockDim.x) {
      const int p = p0 + lane;
      bool head = false;
      if (p < n) {
        const int e = pm[p];
        g.members[gbase + p] = S.V[e];
        if (g.okeys) g.okeys[gbase + p] = K[e];
        head = (p == 0) || K[pm[p - 1]] != K[e];
      }
      const uint32_t hw = __ballot_sync(0xffffffffu, head);
      if (lane == 0) S.hb[p0 >> 5] = hw;
    }
    __syncthreads();
    store_heads(g.head, S.hb, gbase, n, threadIdx.x, blockDim.x);
    __syncthreads();
  }
}

// ============================================================ big tier
__global__ void __launch_bounds__(1024) big_kernel(const __grid_constant__ GroupArgs g) {
  const uint32_t nbig = *g.big_count;
  for (uint32_t li = blockIdx.x; li < nbig; li += gridDim.x) {
    const int64_t q = g.big_list[li];
    int64_t sb, n;
    bucket_extent(g, q, sb, n);
    uint64_t *K = g.bkeys + sb;
    uint32_t *V = g.bvals + sb;
    int64_t M = 1;
    while (M < n) M <<= 1;
    for (int64_t k = 2; k <= M; k <<= 1) {
      for (int64_t jj = k >> 1; jj > 0; jj >>= 1) {
        for (int64_t t = threadIdx.x; t < (M >> 1); t += blockDim.x) {
          const int64_t i = ((t & ~(jj - 1)) << 1) | (t & (jj - 1));
          const int64_t l = (jj == (k >> 1)) ? (i ^ (k - 1)) : (i + jj);
          if (l < n) {
            const uint64_t ka = K[i], kb = K[l];
            const uint32_t va = V[i], vb = V[l];
            if (pair_less(kb, vb, ka, va)) {
              K[i] = kb; K[l] = ka;
              V[i] = vb; V[l] = va;
            }
          }
        }
        __syncthreads();
      }
    }
    const int64_t gbase = g.plan.seg[0] + sb;
    for (int64_t p = threadIdx.x; p < n; p += blockDim.x) {
      g.members[gbase + p] = V[p];
      if (g.okeys) g.okeys[gbase + p] = K[p];
    }
    const int64_t w0 = gbase >> 5, w1 = (gbase + n - 1) >> 5;
    for (int64_t w = w0 + threadIdx.x; w <= w1; w += blockDim.x) {
      uint32_t bits = 0;
      const int64_t lo = max(gbase, w << 5), hi = min(gbase + n, (w << 5) + 32);
      for (int64_t gp = lo; gp < hi; ++gp) {
        const int64_t p = gp - gbase;
        if (p == 0 || K[p] != K[p - 1]) bits |= 1u << (gp & 31);
      }
      if (lo == (w << 5) && hi == (w << 5) + 32) g.head[w] = bits;
      else if (bits) atomicOr(&g.head[w], bits);
    }
    __syncthreads();
  }
}

}  // namespace

int64_t group_local_capacity() { return kLocalCap; }

cudaError_t group_local(const GroupArgs &g, int num_sms, cudaStream_t st) {
  const int64_t nq = (int64_t)g.plan.c * g.plan.nbins;
  if (nq == 0) return cudaSuccess;
  // warp tier over all buckets
  {
    const size_t smem = sizeof(WarpSmem) * kWWarps;
    const int bk = (g.plan.bits == 18 || g.plan.bits == 16 || g.plan.bits == 15) ? g.plan.bits : 0;
    // default: atomic placements + full-order verification (SG_LOCAL_ATOMIC=0:
    // the match-based stable placements, key-only tie check)
    // (forced on when the splits rank atomically: only the verifying tier
    // repairs members that arrive out of generator order)
    static const bool atom = [] {
      const char *e = getenv("SG_LOCAL_ATOMIC");
      return !(e && atoi(e) == 0) || split_atomic() > 0;
    }();
    const void *fn = nullptr;
    switch (bk * 2 + (atom ? 1 : 0)) {
#define SG_WL(B, A) case B * 2 + A: fn = (const void *)warp_local_kernel<B, A>; break;
      SG_WL(18, 1) SG_WL(18, 0) SG_WL(16, 1) SG_WL(16, 0) SG_WL(15, 1) SG_WL(15, 0)
      SG_WL(0, 1) SG_WL(0, 0)
#undef SG_WL
    }
    cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    int per_sm = 0;
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, kWWarps * 32, smem);
    if (e != cudaSuccess) return e;
    per_sm = std::max(per_sm, 1);
    const int64_t want = (nq + kWWarps - 1) / kWWarps;
    const int grid = (int)std::min<int64_t>((int64_t)num_sms * per_sm, want);
    void *args[] = {(void *)&g};
    if ((e = cudaLaunchKernel(fn, dim3(grid), dim3(kWWarps * 32), args, smem, st)) != cudaSuccess) return e;
    ++g_launches;
    if ((e = cudaGetLastError()) != cudaSuccess) return e;
  }
  // CTA tier over the mid list (length read on the device)
  {
    // SG_LOCAL_CTA_ATOMIC=1 (A/B): atomic placements (parity-green; measured
    // slower on the 640M-edge config, whose level-II buckets all take this
    // tier: local2 533.6 vs 521.1 ms)
    static const bool cat = [] {
      const char *e = getenv("SG_LOCAL_CTA_ATOMIC");
      return e && atoi(e) != 0;
    }();
    const size_t smem = sizeof(LocalSmem);
    const void *fn = cat ? (const void *)local_kernel<true> : (const void *)local_kernel<false>;
    cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    if (cat) local_kernel<true><<<num_sms * 2, kLThreads, smem, st>>>(g);
    else local_kernel<false><<<num_sms * 2, kLThreads, smem, st>>>(g);
    ++g_launches;
    if ((e = cudaGetLastError()) != cudaSuccess) return e;
  }
  // big tier (length read on the device)
  return group_big(g, num_sms, st);
}

cudaError_t group_big(const GroupArgs &g, int num_sms, cudaStream_t st) {
  big_kernel<<<num_sms, 1024, 0, st>>>(g);
  ++g_launches;
  return cudaGetLastError();
}

}  // namespace sg
