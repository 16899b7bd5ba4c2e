// kernels_sort.cu — per-trial grouping of <shingle, generator> pairs
// ("a sorting is done to gather all vertices that generated each shingle ...
// once for each random trial", AMB-5), third design
// (DESIGN.md §6.2).  The keys are fmix(id): uniformly spread 64-bit values,
// so a partition by key bits gives near-equal buckets, and the canonical
// order (key, member) is restored inside each small bucket, not carried by
// stable passes:
//
//   1. hist    : per (trial, coarse bin) totals, bin = top B1 <= 11 key bits
//                (shared-memory histogram of 8 chunks per CTA, one global
//                add per bin and flush) -> bucket starts by a scan;
//   2. scatter : one 8K-pair chunk per CTA step: chunk histogram in shared
//                memory, one global fetch-add per bin reserves the chunk's
//                runs in the bucket, pairs placed bin-major in shared memory
//                and written out as contiguous runs (coalesced).  No
//                ordering inside a bucket;
//   3. bucket  : one 1024-thread CTA per coarse bucket (~20K pairs on the 2M
//                graph's level II): counting sort by the next F <= 14 key
//                bits (shared-memory counters, the pairs placed in an
//                L2-resident per-CTA scratch), then every fine bucket (~1-2
//                pairs) is sorted by (key, member) where it lies - by the
//                thread that owns it (<= 8 pairs, registers), by a warp (<=
//                256, shared-memory bitonic) or by the CTA (more, bitonic in
//                the scratch) - and its members are written to their final
//                positions with one head bit per group start.  Coarse
//                buckets above the capacity (a group of tens of thousands of
//                generators) go to big_kernel (kernels_local.cu).
// The result is the oracle's canonical order (AMB-19) whatever order the
// atomics placed the pairs in: (key, member) is a strict total order inside a
// trial (members are unique).
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

constexpr int kHT = 1024;                 // histogram threads
constexpr int kHPer = 8;                  // chunks per histogram CTA
constexpr int kAT = 512;                  // scatter threads
constexpr int kChunkA = 8192;             // pairs per chunk
constexpr int kAPer = kChunkA / kAT;      // 16
constexpr int kMaxB1 = 11;                // coarse bits
constexpr int kMaxBins = 1 << kMaxB1;
constexpr int kBT = 1024;                 // bucket-sort threads
constexpr int kBW = kBT / 32;
constexpr int kMaxF = 14;                 // fine bits
constexpr int kBCap = 65536;              // largest coarse bucket sorted by a CTA
constexpr int kSmall = 8;                 // fine buckets sorted in registers
constexpr int kWarpBuf = 256;             // fine buckets sorted by a warp
constexpr int kMidMax = 4096;             // (unused)
// fine buckets with 2.. pairs, listed per size class (region sizes per coarse bucket)
constexpr int kL2 = 4096, kL4 = 2048, kL8 = 1024, kLW = 1024, kLM = 256;
constexpr int kLTot = kL2 + kL4 + kL8 + kLW + kLM;
constexpr int kBigMax = 64;               // CTA-sorted fine buckets listed per coarse bucket

__device__ __forceinline__ uint32_t top_bits(uint64_t key, int B) {
  return B ? (uint32_t)(key >> (64 - B)) : 0u;
}

// F key bits starting B bits below the MSB
__device__ __forceinline__ uint32_t fine_of(uint64_t key, int B, int F) {
  return F ? (uint32_t)((key << B) >> (64 - F)) : 0u;
}

__device__ __forceinline__ uint32_t val_at3(const GroupArgs &g, int64_t in_idx, int64_t i) {
  if (g.vals) return g.vals[in_idx];
  if (g.rowid) return g.rowid[i];
  return g.val_base + (uint32_t)i;
}

// ---- 1. coarse histogram ------------------------------------------------------
// bsize1[j][b] += count of bin b in the CTA's chunks of trial j (zeroed by the
// caller); chunks of one trial are consecutive in the chunk table.
__global__ void __launch_bounds__(kHT) hist_c_kernel(const __grid_constant__ GroupArgs g) {
  __shared__ uint32_t h[kMaxBins];
  const int B = g.plan.bits1;
  const int nb = 1 << B;
  const int64_t k0 = (int64_t)blockIdx.x * kHPer;
  const int64_t k1 = min(k0 + kHPer, g.plan.nchunks);
  for (int i = threadIdx.x; i < nb; i += kHT) h[i] = 0;
  __syncthreads();
  int j = g.plan.chunk_trial[k0];
  for (int64_t k = k0; k < k1; ++k) {
    const int jk = g.plan.chunk_trial[k];
    if (jk != j) {                                   // trial boundary: flush
      __syncthreads();
      for (int b = threadIdx.x; b < nb; b += kHT) {
        if (h[b]) atomicAdd(&g.bsize1[(int64_t)j * nb + b], h[b]);
        h[b] = 0;
      }
      __syncthreads();
      j = jk;
    }
    const uint64_t *__restrict__ keys = g.keys + g.plan.chunk_in0[k];
    const int len = g.plan.chunk_len[k];
    int i = threadIdx.x;
    for (; i + 3 * kHT < len; i += 4 * kHT) {
      const uint64_t a = keys[i], b = keys[i + kHT], c = keys[i + 2 * kHT], d = keys[i + 3 * kHT];
      atomicAdd(&h[top_bits(a, B)], 1u);
      atomicAdd(&h[top_bits(b, B)], 1u);
      atomicAdd(&h[top_bits(c, B)], 1u);
      atomicAdd(&h[top_bits(d, B)], 1u);
    }
    for (; i < len; i += kHT) atomicAdd(&h[top_bits(keys[i], B)], 1u);
  }
  __syncthreads();
  for (int b = threadIdx.x; b < nb; b += kHT)
    if (h[b]) atomicAdd(&g.bsize1[(int64_t)j * nb + b], h[b]);
}

// cursor[j][b] = bstart1[j][b] (the scatter's running reservation points)
__global__ void copy_u32_kernel(const uint32_t *__restrict__ a, uint32_t *__restrict__ b, int64_t n) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x)
    b[i] = a[i];
}

// ---- 2. coarse scatter ----------------------------------------------------------
struct ASmem {
  uint64_t K[kChunkA];
  uint16_t I[kChunkA];          // chunk index of the pair at a placed slot
  uint32_t cur[kMaxBins];       // counts -> local cursors
  uint32_t off[kMaxBins];       // bucket position - local position (u32 wrap)
  int64_t ws[33];
};

__global__ void __launch_bounds__(kAT, 2) scatter_c_kernel(const __grid_constant__ GroupArgs g) {
  extern __shared__ __align__(16) unsigned char smraw[];
  ASmem &S = *reinterpret_cast<ASmem *>(smraw);
  const int B = g.plan.bits1;
  const int nb = 1 << B;
  constexpr int kBinsPer = kMaxBins / kAT;     // 4
  uint64_t kk[kAPer];
  auto load = [&](int64_t k) {
    const int64_t in0 = g.plan.chunk_in0[k];
    const int len = g.plan.chunk_len[k];
#pragma unroll
    for (int u = 0; u < kAPer; ++u) {
      const int i = threadIdx.x + u * kAT;
      kk[u] = i < len ? g.keys[in0 + i] : 0ull;
    }
  };
  int64_t k = blockIdx.x;
  if (k < g.plan.nchunks) load(k);
  while (k < g.plan.nchunks) {
    const int j = g.plan.chunk_trial[k];
    const int64_t in0 = g.plan.chunk_in0[k], i0 = g.plan.chunk_i0[k];
    const int len = g.plan.chunk_len[k];
    const int64_t sseg = g.plan.seg[j] - g.plan.seg[0];
    for (int b = threadIdx.x; b < nb; b += kAT) S.cur[b] = 0;
    __syncthreads();
#pragma unroll
    for (int u = 0; u < kAPer; ++u)
      if (threadIdx.x + u * kAT < len) atomicAdd(&S.cur[top_bits(kk[u], B)], 1u);
    __syncthreads();
    {
      // local starts (exclusive scan, kBinsPer consecutive bins per thread) and
      // the chunk's run in each bucket (one global reservation per bin)
      const int b0 = threadIdx.x * kBinsPer;
      uint32_t c[kBinsPer], s = 0;
#pragma unroll
      for (int x = 0; x < kBinsPer; ++x) {
        c[x] = b0 + x < nb ? S.cur[b0 + x] : 0u;
        s += c[x];
      }
      int64_t tot;
      uint32_t run = (uint32_t)block_excl_scan<int64_t>((int64_t)s, S.ws, &tot);
#pragma unroll
      for (int x = 0; x < kBinsPer; ++x) {
        if (b0 + x < nb) {
          S.cur[b0 + x] = run;
          if (c[x]) {
            const uint32_t gpos = atomicAdd(&g.gcur[(int64_t)j * nb + b0 + x], c[x]);
            S.off[b0 + x] = gpos - run;
          }
          run += c[x];
        }
      }
    }
    __syncthreads();
#pragma unroll
    for (int u = 0; u < kAPer; ++u) {
      const int i = threadIdx.x + u * kAT;
      if (i < len) {
        const uint32_t p = atomicAdd(&S.cur[top_bits(kk[u], B)], 1u);
        S.K[p] = kk[u];
        S.I[p] = (uint16_t)i;
      }
    }
    __syncthreads();
    const int64_t kn = k + gridDim.x;
    if (kn < g.plan.nchunks) load(kn);            // in flight during the stores below
    for (int p = threadIdx.x; p < len; p += kAT) {
      const uint64_t key = S.K[p];
      const uint32_t o = S.off[top_bits(key, B)] + (uint32_t)p;
      const int e = S.I[p];
      g.akeys[sseg + o] = key;
      g.avals[sseg + o] = val_at3(g, in0 + e, i0 + e);
    }
    __syncthreads();
    k = kn;
  }
}

// ---- 3. per coarse bucket: counting sort by the fine bits + small sorts ----------
constexpr int kBigSmem = 8192;            // fine buckets sorted by the CTA in shared memory

struct BSmem {
  uint32_t cur[1 << kMaxF];              // fine counts -> starts -> ends
  uint32_t hb[kBCap / 32 + 2];           // head bits of the bucket
  union {
    struct {                             // per-warp sort buffers (9..256 pairs)
      uint64_t k[kBW][kWarpBuf];
      uint32_t v[kBW][kWarpBuf];
    } w;
    struct {                             // one CTA-wide sort (257..8192 pairs)
      uint64_t k[kBigSmem];
      uint32_t v[kBigSmem];
    } c;
  } buf;
  uint32_t lst[kLTot];                   // fine buckets by size class: 2, 3-4, 5-8, 9-32, 33-256
  uint32_t big[kBigMax];
  uint32_t ncls[5], nbig;
  int64_t ws[33];
};
static_assert(sizeof(uint64_t) * kBW * kWarpBuf + sizeof(uint32_t) * kBW * kWarpBuf ==
                  sizeof(uint64_t) * kBigSmem + sizeof(uint32_t) * kBigSmem,
              "the two sort buffers share their storage");

__device__ __forceinline__ void cswap(uint64_t &ka, uint32_t &va, uint64_t &kb, uint32_t &vb) {
  if (pair_less(kb, vb, ka, va)) {
    const uint64_t tk = ka;
    ka = kb;
    kb = tk;
    const uint32_t tv = va;
    va = vb;
    vb = tv;
  }
}

// Writes the sorted run (k[0..m), v[0..m)) of fine bucket [s, s+m): members
// and a head bit at every key change (the run's first pair always starts a
// group: the previous fine bucket has other key bits).
__device__ __forceinline__ void emit_one(const GroupArgs &g, BSmem &S, int64_t gbase, uint32_t p,
                                         uint64_t key, uint32_t val, bool head) {
  g.members[gbase + p] = val;
  if (g.okeys) g.okeys[gbase + p] = key;
  if (head) atomicOr(&S.hb[p >> 5], 1u << (p & 31));
}

__global__ void __launch_bounds__(kBT, 1) bucket_c_kernel(const __grid_constant__ GroupArgs g) {
  extern __shared__ __align__(16) unsigned char smraw[];
  BSmem &S = *reinterpret_cast<BSmem *>(smraw);
  const int B = g.plan.bits1;
  const int F = g.plan.fine_bits;
  const int nf = 1 << F;
  const int cap = g.plan.local_cap;
  const int64_t nq = (int64_t)g.plan.c * g.plan.nb1;
  const int64_t obase = g.plan.seg[0];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  uint64_t *__restrict__ SK = g.bkeys + (int64_t)blockIdx.x * kBCap;     // this CTA's scratch
  uint32_t *__restrict__ SV = g.bvals + (int64_t)blockIdx.x * kBCap;
  for (int64_t q = blockIdx.x; q < nq; q += gridDim.x) {
    const int64_t n64 = g.bsize1[q];
    if (n64 == 0) continue;
    const int j = (int)(q / g.plan.nb1);
    const int64_t sb = (g.plan.seg[j] - g.plan.seg[0]) + g.bstart1[q];
    if (n64 > cap) {
      if (threadIdx.x == 0) g.big_list[atomicAdd(g.big_count, 1u)] = (uint32_t)q;
      continue;
    }
    const int n = (int)n64;
    const uint64_t *__restrict__ Kg = g.akeys + sb;
    const uint32_t *__restrict__ Vg = g.avals + sb;
    const int64_t gbase = obase + sb;
    for (int i = threadIdx.x; i < nf; i += kBT) S.cur[i] = 0;
    for (int i = threadIdx.x; i < ((n + 31) >> 5) + 1; i += kBT) S.hb[i] = 0;
    if (threadIdx.x < 5) S.ncls[threadIdx.x] = 0;
    if (threadIdx.x == 0) S.nbig = 0;
    __syncthreads();
    // fine histogram
    {
      int i = threadIdx.x;
      for (; i + 3 * kBT < n; i += 4 * kBT) {
        const uint64_t a = Kg[i], b = Kg[i + kBT], c = Kg[i + 2 * kBT], d = Kg[i + 3 * kBT];
        atomicAdd(&S.cur[fine_of(a, B, F)], 1u);
        atomicAdd(&S.cur[fine_of(b, B, F)], 1u);
        atomicAdd(&S.cur[fine_of(c, B, F)], 1u);
        atomicAdd(&S.cur[fine_of(d, B, F)], 1u);
      }
      for (; i < n; i += kBT) atomicAdd(&S.cur[fine_of(Kg[i], B, F)], 1u);
    }
    __syncthreads();
    {
      // exclusive scan: thread t owns nf / kBT consecutive fine buckets
      const int per = (nf + kBT - 1) / kBT;
      const int f0 = threadIdx.x * per;
      uint32_t s = 0;
      for (int x = 0; x < per; ++x)
        if (f0 + x < nf) s += S.cur[f0 + x];
      int64_t tot;
      uint32_t run = (uint32_t)block_excl_scan<int64_t>((int64_t)s, S.ws, &tot);
      for (int x = 0; x < per; ++x)
        if (f0 + x < nf) {
          const uint32_t v = S.cur[f0 + x];
          S.cur[f0 + x] = run;
          run += v;
        }
    }
    __syncthreads();
    // counting-sort placement into the scratch (cur[f] ends as the end of f)
    {
      int i = threadIdx.x;
      for (; i + kBT < n; i += 2 * kBT) {
        const uint64_t a = Kg[i], b = Kg[i + kBT];
        const uint32_t va = Vg[i], vb = Vg[i + kBT];
        const uint32_t pa = atomicAdd(&S.cur[fine_of(a, B, F)], 1u);
        const uint32_t pb = atomicAdd(&S.cur[fine_of(b, B, F)], 1u);
        SK[pa] = a;
        SV[pa] = va;
        SK[pb] = b;
        SV[pb] = vb;
      }
      if (i < n) {
        const uint64_t a = Kg[i];
        const uint32_t pa = atomicAdd(&S.cur[fine_of(a, B, F)], 1u);
        SK[pa] = a;
        SV[pa] = Vg[i];
      }
    }
    __syncthreads();
    // single-pair fine buckets (most of them): one coalesced pass over the
    // scratch, each pair is already at its final position
    for (int p0 = 0; p0 < n; p0 += kBT) {
      const int p = p0 + threadIdx.x;
      bool single = false;
      if (p < n) {
        const uint64_t key = SK[p];
        const uint32_t f = fine_of(key, B, F);
        const uint32_t s = f ? S.cur[f - 1] : 0u;
        if (S.cur[f] - s == 1u) {
          single = true;
          g.members[gbase + p] = SV[p];
          if (g.okeys) g.okeys[gbase + p] = key;
        }
      }
      const uint32_t hw = __ballot_sync(0xffffffffu, single);
      if (lane == 0 && hw) atomicOr(&S.hb[p >> 5], hw);
    }
    // fine buckets of >= 2 pairs (a group, or keys sharing the fine bits):
    // listed by size class, then sorted by (key, member) with every lane busy
    for (int f = threadIdx.x; f < nf; f += kBT) {
      const uint32_t e = S.cur[f];
      const uint32_t s = f ? S.cur[f - 1] : 0u;
      const uint32_t m = e - s;
      if (m <= 1) continue;
      const int c = m == 2 ? 0 : m <= 4 ? 1 : m <= 8 ? 2 : m <= 32 ? 3 : m <= (uint32_t)kWarpBuf ? 4 : 5;
      bool listed = false;
      if (c < 5) {
        const int base = c == 0 ? 0 : c == 1 ? kL2 : c == 2 ? kL2 + kL4 : c == 3 ? kL2 + kL4 + kL8
                                                                        : kL2 + kL4 + kL8 + kLW;
        const int cap = c == 0 ? kL2 : c == 1 ? kL4 : c == 2 ? kL8 : c == 3 ? kLW : kLM;
        const uint32_t t = atomicAdd(&S.ncls[c], 1u);
        if (t < (uint32_t)cap) {
          S.lst[base + t] = (uint32_t)f;
          listed = true;
        }
      }
      if (!listed) {
        const uint32_t u = atomicAdd(&S.nbig, 1u);
        if (u < kBigMax) S.big[u] = (uint32_t)f;
      }
    }
    __syncthreads();
    {
      // 2 pairs: one compare-exchange
      const int n2 = min(S.ncls[0], (uint32_t)kL2);
      for (int x = threadIdx.x; x < n2; x += kBT) {
        const int f = S.lst[x];
        const uint32_t s = f ? S.cur[f - 1] : 0u;
        uint64_t k0 = SK[s], k1 = SK[s + 1];
        uint32_t v0 = SV[s], v1 = SV[s + 1];
        cswap(k0, v0, k1, v1);
        emit_one(g, S, gbase, s, k0, v0, true);
        emit_one(g, S, gbase, s + 1, k1, v1, k1 != k0);
      }
      // 3-4 pairs: Batcher network on 4
      const int n4 = min(S.ncls[1], (uint32_t)kL4);
      for (int x = threadIdx.x; x < n4; x += kBT) {
        const int f = S.lst[kL2 + x];
        const uint32_t s = f ? S.cur[f - 1] : 0u;
        const uint32_t m = S.cur[f] - s;
        uint64_t k[4];
        uint32_t v[4];
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          const bool in = (uint32_t)i < m;
          k[i] = in ? SK[s + i] : ~0ull;
          v[i] = in ? SV[s + i] : ~0u;
        }
        cswap(k[0], v[0], k[1], v[1]); cswap(k[2], v[2], k[3], v[3]);
        cswap(k[0], v[0], k[2], v[2]); cswap(k[1], v[1], k[3], v[3]);
        cswap(k[1], v[1], k[2], v[2]);
#pragma unroll
        for (int i = 0; i < 4; ++i)
          if ((uint32_t)i < m) emit_one(g, S, gbase, s + i, k[i], v[i], i == 0 || k[i] != k[i - 1]);
      }
      // 5-8 pairs: Batcher odd-even merge network on 8 (pads sort last:
      // members < 2^32 - 1)
      const int n8 = min(S.ncls[2], (uint32_t)kL8);
      for (int x = threadIdx.x; x < n8; x += kBT) {
        const int f = S.lst[kL2 + kL4 + x];
        const uint32_t s = f ? S.cur[f - 1] : 0u;
        const uint32_t m = S.cur[f] - s;
        uint64_t k[kSmall];
        uint32_t v[kSmall];
#pragma unroll
        for (int i = 0; i < kSmall; ++i) {
          const bool in = (uint32_t)i < m;
          k[i] = in ? SK[s + i] : ~0ull;
          v[i] = in ? SV[s + i] : ~0u;
        }
        cswap(k[0], v[0], k[1], v[1]); cswap(k[2], v[2], k[3], v[3]);
        cswap(k[4], v[4], k[5], v[5]); cswap(k[6], v[6], k[7], v[7]);
        cswap(k[0], v[0], k[2], v[2]); cswap(k[1], v[1], k[3], v[3]);
        cswap(k[4], v[4], k[6], v[6]); cswap(k[5], v[5], k[7], v[7]);
        cswap(k[1], v[1], k[2], v[2]); cswap(k[5], v[5], k[6], v[6]);
        cswap(k[0], v[0], k[4], v[4]); cswap(k[1], v[1], k[5], v[5]);
        cswap(k[2], v[2], k[6], v[6]); cswap(k[3], v[3], k[7], v[7]);
        cswap(k[2], v[2], k[4], v[4]); cswap(k[3], v[3], k[5], v[5]);
        cswap(k[1], v[1], k[2], v[2]); cswap(k[3], v[3], k[4], v[4]);
        cswap(k[5], v[5], k[6], v[6]);
#pragma unroll
        for (int i = 0; i < kSmall; ++i)
          if ((uint32_t)i < m) emit_one(g, S, gbase, s + i, k[i], v[i], i == 0 || k[i] != k[i - 1]);
      }
      // 9-32 pairs: a warp each, one pair per lane, bitonic by shuffles
      const int nw32 = min(S.ncls[3], (uint32_t)kLW);
      for (int x = w; x < nw32; x += kBW) {
        const int f = S.lst[kL2 + kL4 + kL8 + x];
        const uint32_t s = f ? S.cur[f - 1] : 0u;
        const uint32_t m = S.cur[f] - s;
        const bool in = (uint32_t)lane < m;
        uint64_t k = in ? SK[s + lane] : ~0ull;
        uint32_t v = in ? SV[s + lane] : ~0u;
#pragma unroll
        for (int kk = 2; kk <= 32; kk <<= 1)
#pragma unroll
          for (int jj = kk >> 1; jj > 0; jj >>= 1) {
            const uint64_t ok = __shfl_xor_sync(0xffffffffu, k, jj);
            const uint32_t ov = __shfl_xor_sync(0xffffffffu, v, jj);
            const bool up = (lane & kk) == 0, lower = (lane & jj) == 0;
            const bool other_less = pair_less(ok, ov, k, v);
            if ((lower == up) ? other_less : !other_less) {
              k = ok;
              v = ov;
            }
          }
        const uint64_t prev = __shfl_up_sync(0xffffffffu, k, 1);
        if (in) emit_one(g, S, gbase, s + lane, k, v, lane == 0 || prev != k);
      }
    }
    // 33..256 pairs: a warp each, bitonic sort in its shared-memory buffer
    const uint32_t nmid = min(S.ncls[4], (uint32_t)kLM);
    for (uint32_t x = w; x < nmid; x += kBW) {
      const int f = S.lst[kL2 + kL4 + kL8 + kLW + x];
      const uint32_t e = S.cur[f];
      const uint32_t s = f ? S.cur[f - 1] : 0u;
      const int m = (int)(e - s);
      int M = 64;
      while (M < m) M <<= 1;
      for (int i = lane; i < M; i += 32) {
        S.buf.w.k[w][i] = i < m ? SK[s + i] : ~0ull;
        S.buf.w.v[w][i] = i < m ? SV[s + i] : ~0u;
      }
      __syncwarp();
      for (int kk = 2; kk <= M; kk <<= 1)
        for (int jj = kk >> 1; jj > 0; jj >>= 1) {
          for (int t = lane; t < (M >> 1); t += 32) {
            const int a = ((t & ~(jj - 1)) << 1) | (t & (jj - 1));
            const int b = (jj == (kk >> 1)) ? (a ^ (kk - 1)) : (a + jj);
            uint64_t ka = S.buf.w.k[w][a], kb = S.buf.w.k[w][b];
            uint32_t va = S.buf.w.v[w][a], vb = S.buf.w.v[w][b];
            if (pair_less(kb, vb, ka, va)) {
              S.buf.w.k[w][a] = kb;
              S.buf.w.k[w][b] = ka;
              S.buf.w.v[w][a] = vb;
              S.buf.w.v[w][b] = va;
            }
          }
          __syncwarp();
        }
      for (int i = lane; i < m; i += 32)
        emit_one(g, S, gbase, s + i, S.buf.w.k[w][i], S.buf.w.v[w][i], i == 0 || S.buf.w.k[w][i] != S.buf.w.k[w][i - 1]);
      __syncwarp();
    }
    // larger fine buckets (a group of hundreds+ generators): the whole CTA,
    // bitonic in shared memory (<= 8192 pairs) or in the scratch; more than
    // kBigMax of them: the whole coarse bucket in one sort (pathological)
    __syncthreads();
    const uint32_t nbig = S.nbig;
    const uint32_t nb_lists = nbig > (uint32_t)kBigMax ? 1u : nbig;
    for (uint32_t x = 0; x < nb_lists; ++x) {
      uint32_t s, m;
      if (nbig > (uint32_t)kBigMax) {
        s = 0;
        m = (uint32_t)n;
      } else {
        const int f = S.big[x];
        s = f ? S.cur[f - 1] : 0u;
        m = S.cur[f] - s;
      }
      uint32_t M = 1;
      while (M < m) M <<= 1;
      const bool sm = M <= (uint32_t)kBigSmem;
      if (sm) {
        for (uint32_t i = threadIdx.x; i < M; i += kBT) {
          S.buf.c.k[i] = i < m ? SK[s + i] : ~0ull;
          S.buf.c.v[i] = i < m ? SV[s + i] : ~0u;
        }
        __syncthreads();
      }
      for (uint32_t kk = 2; kk <= M; kk <<= 1)
        for (uint32_t jj = kk >> 1; jj > 0; jj >>= 1) {
          for (uint32_t t = threadIdx.x; t < (M >> 1); t += kBT) {
            const uint32_t a = ((t & ~(jj - 1)) << 1) | (t & (jj - 1));
            const uint32_t b = (jj == (kk >> 1)) ? (a ^ (kk - 1)) : (a + jj);
            if (sm) {
              const uint64_t ka = S.buf.c.k[a], kb = S.buf.c.k[b];
              const uint32_t va = S.buf.c.v[a], vb = S.buf.c.v[b];
              if (pair_less(kb, vb, ka, va)) {
                S.buf.c.k[a] = kb;
                S.buf.c.k[b] = ka;
                S.buf.c.v[a] = vb;
                S.buf.c.v[b] = va;
              }
            } else if (b < m) {
              const uint64_t ka = SK[s + a], kb = SK[s + b];
              const uint32_t va = SV[s + a], vb = SV[s + b];
              if (pair_less(kb, vb, ka, va)) {
                SK[s + a] = kb;
                SK[s + b] = ka;
                SV[s + a] = vb;
                SV[s + b] = va;
              }
            }
          }
          __syncthreads();
        }
      for (uint32_t i = threadIdx.x; i < m; i += kBT) {
        const uint64_t key = sm ? S.buf.c.k[i] : SK[s + i];
        const uint64_t prev = i == 0 ? 0ull : (sm ? S.buf.c.k[i - 1] : SK[s + i - 1]);
        emit_one(g, S, gbase, s + i, key, sm ? S.buf.c.v[i] : SV[s + i], i == 0 || prev != key);
      }
      __syncthreads();
    }
    // head words of the bucket into the global bit array (boundary words OR-ed)
    {
      const int64_t w0 = gbase >> 5, w1 = (gbase + n - 1) >> 5;
      const int off = (int)(gbase & 31);
      const int nw = (n + 31) >> 5;
      for (int64_t wd = w0 + threadIdx.x; wd <= w1; wd += kBT) {
        const int k = (int)(wd - w0);
        uint32_t bits;
        if (off == 0) {
          bits = k < nw ? S.hb[k] : 0u;
        } else {
          const uint32_t lo = (k >= 1 && k - 1 < nw) ? S.hb[k - 1] : 0u;
          const uint32_t hi = k < nw ? S.hb[k] : 0u;
          bits = (lo >> (32 - off)) | (hi << off);
        }
        const int64_t lo_pos = wd << 5, hi_pos = lo_pos + 32;
        if (lo_pos >= gbase && hi_pos <= gbase + n) g.head[wd] = bits;
        else if (bits) atomicOr(&g.head[wd], bits);
      }
    }
    __syncthreads();
  }
}

}  // namespace

int64_t group_c_chunk_pairs() { return kChunkA; }
int32_t group_c_local_cap() { return kBCap; }
int64_t group_c_scratch_pairs(int num_sms) { return (int64_t)num_sms * kBCap; }

void group_c_bits(int64_t maxseg, int32_t *bits1, int32_t *fine_bits) {
  // coarse buckets of ~20K pairs on average (a CTA sorts up to 64K), fine
  // buckets of ~1-2 pairs; test hook SG_GROUP_TARGET: smaller coarse buckets
  const char *e = getenv("SG_GROUP_TARGET");
  int64_t target = e ? atoll(e) : 24576;
  if (target <= 0) target = 24576;
  int b = 0;
  while ((maxseg >> b) > target && b < kMaxB1) ++b;
  const int64_t avg = (maxseg >> b) + 1;
  int f = 0;
  while ((avg >> f) > 1 && f < kMaxF) ++f;
  *bits1 = b;
  *fine_bits = f;
}

cudaError_t group_c_hist(const GroupArgs &a, int num_sms, cudaStream_t st) {
  (void)num_sms;
  if (a.plan.nchunks == 0) return cudaSuccess;
  const int B = a.plan.bits1;
  if (B < 0 || B > kMaxB1) return cudaErrorInvalidValue;
  const int64_t nb = (int64_t)1 << B;
  cudaError_t e = cudaMemsetAsync(a.bsize1, 0, (size_t)(a.plan.c * nb) * 4, st);
  if (e != cudaSuccess) return e;
  const unsigned grid = (unsigned)((a.plan.nchunks + kHPer - 1) / kHPer);
  hist_c_kernel<<<grid, kHT, 0, st>>>(a);
  ++g_launches;
  if ((e = cudaGetLastError()) != cudaSuccess) return e;
  // bucket starts (exclusive scan per trial) and the scatter's cursors
  GroupArgs o = a;
  o.plan.nb1 = nb;
  if ((e = group_binscan(o, st)) != cudaSuccess) return e;
  const int64_t tot = a.plan.c * nb;
  copy_u32_kernel<<<(unsigned)std::min<int64_t>((tot + 255) / 256, 4096), 256, 0, st>>>(a.bstart1,
                                                                                       a.gcur, tot);
  ++g_launches;
  return cudaGetLastError();
}

cudaError_t group_c_scatter(const GroupArgs &a, int num_sms, cudaStream_t st) {
  if (a.plan.nchunks == 0) return cudaSuccess;
  if (a.plan.bits1 < 0 || a.plan.bits1 > kMaxB1) return cudaErrorInvalidValue;
  const size_t smem = sizeof(ASmem);
  cudaError_t e = cudaFuncSetAttribute(scatter_c_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       (int)smem);
  if (e != cudaSuccess) return e;
  const int grid = (int)std::min<int64_t>((int64_t)num_sms * 2, a.plan.nchunks);
  scatter_c_kernel<<<grid, kAT, smem, st>>>(a);
  ++g_launches;
  return cudaGetLastError();
}

cudaError_t group_c_bucket(const GroupArgs &a0, int num_sms, cudaStream_t st) {
  GroupArgs a = a0;
  if (a.plan.local_cap <= 0 || a.plan.local_cap > kBCap) a.plan.local_cap = kBCap;
  if (a.plan.fine_bits < 0 || a.plan.fine_bits > kMaxF) return cudaErrorInvalidValue;
  const int64_t nq = (int64_t)a.plan.c * a.plan.nb1;
  if (nq == 0) return cudaSuccess;
  const size_t smem = sizeof(BSmem);
  cudaError_t e = cudaFuncSetAttribute(bucket_c_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       (int)smem);
  if (e != cudaSuccess) return e;
  const int grid = (int)std::min<int64_t>(num_sms, nq);
  bucket_c_kernel<<<grid, kBT, smem, st>>>(a);
  ++g_launches;
  if ((e = cudaGetLastError()) != cudaSuccess) return e;
  // coarse buckets above the capacity: global-memory sort in place
  GroupArgs b = a;
  b.bkeys = a.akeys;
  b.bvals = a.avals;
  b.bstart = a.bstart1;
  b.bsize = a.bsize1;
  b.plan.nbins = a.plan.nb1;
  return group_big(b, num_sms, st);
}

}  // namespace sg
