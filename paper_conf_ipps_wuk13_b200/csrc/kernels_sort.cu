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
constexpr int kHPer = 16;                 // chunks per histogram CTA
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
// fine buckets with 2..8 pairs (sorted by a thread) and with more (a warp)
constexpr int kL8 = 8192, kLW = 2048;
constexpr int kBigMax = 256;              // CTA-sorted fine buckets listed per coarse bucket

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
constexpr int kBigSmem = 2048;            // multi-key fine buckets sorted by the CTA in shared memory

struct BSmem {
  uint32_t cur[1 << kMaxF];              // fine counts -> starts -> ends
  uint32_t hb[kBCap / 32 + 2];           // head bits of the bucket
  uint64_t bk[kBigSmem];                 // one CTA-wide sort (rare: several keys, > 8 pairs)
  uint32_t bv[kBigSmem];
  uint32_t l8[kL8];                      // fine buckets of 2..8 pairs
  uint32_t lw[kLW];                      // fine buckets of > 8 pairs
  uint32_t big[kBigMax];
  uint32_t n8, nw, nbig;
  int64_t ws[33];
};

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
    if (threadIdx.x == 0) S.n8 = S.nw = S.nbig = 0;
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
    // fine buckets of >= 2 pairs: almost always ONE group (one key) whose
    // members only need ordering
    for (int f = threadIdx.x; f < nf; f += kBT) {
      const uint32_t e = S.cur[f];
      const uint32_t s = f ? S.cur[f - 1] : 0u;
      const uint32_t m = e - s;
      if (m <= 1) continue;
      bool listed = false;
      if (m <= kSmall) {
        const uint32_t t = atomicAdd(&S.n8, 1u);
        if (t < (uint32_t)kL8) { S.l8[t] = (uint32_t)f; listed = true; }
      } else {
        const uint32_t t = atomicAdd(&S.nw, 1u);
        if (t < (uint32_t)kLW) { S.lw[t] = (uint32_t)f; listed = true; }
      }
      if (!listed) {
        const uint32_t u = atomicAdd(&S.nbig, 1u);
        if (u < kBigMax) S.big[u] = (uint32_t)f;
      }
    }
    __syncthreads();
    {
      // 2..8 pairs, one fine bucket per thread (every lane busy)
      const int n8 = min(S.n8, (uint32_t)kL8);
      for (int x = threadIdx.x; x < n8; x += kBT) {
        const int f = S.l8[x];
        const uint32_t s = f ? S.cur[f - 1] : 0u;
        const uint32_t m = S.cur[f] - s;
        uint64_t k[kSmall];
        uint32_t v[kSmall];
        bool one = true;
#pragma unroll
        for (int i = 0; i < kSmall; ++i) {
          const bool in = (uint32_t)i < m;
          k[i] = in ? SK[s + i] : ~0ull;
          v[i] = in ? SV[s + i] : ~0u;
          one &= !in || k[i] == k[0];
        }
        if (one) {
          // one group: order the members (pads ~0 sort last: members < 2^32 - 1)
#define MS(a, b) { const uint32_t lo = min(v[a], v[b]); v[b] = max(v[a], v[b]); v[a] = lo; }
          if (m == 2) {
            MS(0, 1);
          } else {
            MS(0, 1); MS(2, 3); MS(4, 5); MS(6, 7); MS(0, 2); MS(1, 3); MS(4, 6); MS(5, 7);
            MS(1, 2); MS(5, 6); MS(0, 4); MS(1, 5); MS(2, 6); MS(3, 7); MS(2, 4); MS(3, 5);
            MS(1, 2); MS(3, 4); MS(5, 6);
          }
#undef MS
#pragma unroll
          for (int i = 0; i < kSmall; ++i)
            if ((uint32_t)i < m) emit_one(g, S, gbase, s + i, k[0], v[i], i == 0);
        } else {
          // several keys share the fine bits: Batcher network on (key, member)
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
      }
      // > 8 pairs, a warp each: one key -> members written in place unsorted
      // and the segment listed for the segmented member sort (group_c_segsort);
      // several keys (rare) -> the CTA sort below
      const int nwl = min(S.nw, (uint32_t)kLW);
      for (int x = w; x < nwl; x += kBW) {
        const int f = S.lw[x];
        const uint32_t s = f ? S.cur[f - 1] : 0u;
        const uint32_t m = S.cur[f] - s;
        const uint64_t k0 = SK[s];
        bool one = true;
        for (uint32_t i = lane; i < m; i += 32) one &= SK[s + i] == k0;
        one = __all_sync(0xffffffffu, one);
        if (one) {
          for (uint32_t i = lane; i < m; i += 32) {
            g.members[gbase + s + i] = SV[s + i];
            if (g.okeys) g.okeys[gbase + s + i] = k0;
          }
          if (lane == 0) {
            atomicOr(&S.hb[s >> 5], 1u << (s & 31));
            const unsigned long long t = atomicAdd(g.seg_count, 1ull);
            g.seg_pos[t] = gbase + s;
            g.seg_len[t] = m;
          }
        } else {
          // several keys (a big group + keys sharing its fine bits): key runs in
          // ascending key order, each run's members in place, then ordered
          // (here when short, by the segmented sort when > 8)
          const uint32_t lt = (1u << lane) - 1u;
          uint32_t outp = s;
          uint64_t last = 0;
          bool first = true;
          for (;;) {
            uint64_t km = ~0ull;
            bool any = false;
            for (uint32_t i = lane; i < m; i += 32) {
              const uint64_t kx = SK[s + i];
              if ((first || kx > last) && kx <= km) {
                km = kx;
                any = true;
              }
            }
            if (!__any_sync(0xffffffffu, any)) break;
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) {
              const uint64_t ko = __shfl_xor_sync(0xffffffffu, km, o);
              km = ko < km ? ko : km;
            }
            uint32_t cnt = 0;
            for (uint32_t i0 = 0; i0 < m; i0 += 32) {
              const uint32_t i = i0 + lane;
              const bool sel = i < m && SK[s + i] == km;
              const uint32_t mask = __ballot_sync(0xffffffffu, sel);
              if (sel) {
                const uint32_t pos = outp + cnt + __popc(mask & lt);
                g.members[gbase + pos] = SV[s + i];
                if (g.okeys) g.okeys[gbase + pos] = km;
              }
              cnt += __popc(mask);
            }
            __syncwarp();
            if (lane == 0) {
              atomicOr(&S.hb[outp >> 5], 1u << (outp & 31));
              if (cnt > (uint32_t)kSmall) {
                const unsigned long long t = atomicAdd(g.seg_count, 1ull);
                g.seg_pos[t] = gbase + outp;
                g.seg_len[t] = cnt;
              } else {
                uint32_t *p = g.members + gbase + outp;
                for (uint32_t x = 1; x < cnt; ++x) {
                  const uint32_t e = p[x];
                  int y = (int)x - 1;
                  while (y >= 0 && e < p[y]) { p[y + 1] = p[y]; --y; }
                  p[y + 1] = e;
                }
              }
            }
            __syncwarp();
            outp += cnt;
            last = km;
            first = false;
          }
        }
      }
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
          S.bk[i] = i < m ? SK[s + i] : ~0ull;
          S.bv[i] = i < m ? SV[s + i] : ~0u;
        }
        __syncthreads();
      }
      for (uint32_t kk = 2; kk <= M; kk <<= 1)
        for (uint32_t jj = kk >> 1; jj > 0; jj >>= 1) {
          for (uint32_t t = threadIdx.x; t < (M >> 1); t += kBT) {
            const uint32_t a = ((t & ~(jj - 1)) << 1) | (t & (jj - 1));
            const uint32_t b = (jj == (kk >> 1)) ? (a ^ (kk - 1)) : (a + jj);
            if (sm) {
              const uint64_t ka = S.bk[a], kb = S.bk[b];
              const uint32_t va = S.bv[a], vb = S.bv[b];
              if (pair_less(kb, vb, ka, va)) {
                S.bk[a] = kb;
                S.bk[b] = ka;
                S.bv[a] = vb;
                S.bv[b] = va;
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
        const uint64_t key = sm ? S.bk[i] : SK[s + i];
        const uint64_t prev = i == 0 ? 0ull : (sm ? S.bk[i - 1] : SK[s + i - 1]);
        emit_one(g, S, gbase, s + i, key, sm ? S.bv[i] : SV[s + i], i == 0 || prev != key);
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

// ---- 4. segmented member sort of one-key fine buckets of > 8 members --------
constexpr int kSWT = 256;
constexpr int kSWBuf = 1024;             // members per warp buffer
constexpr int kSCBuf = 16384;            // members per CTA buffer

__device__ __forceinline__ void bitonic32_u32(uint32_t &v, int lane) {
#pragma unroll
  for (int kk = 2; kk <= 32; kk <<= 1)
#pragma unroll
    for (int jj = kk >> 1; jj > 0; jj >>= 1) {
      const uint32_t o = __shfl_xor_sync(0xffffffffu, v, jj);
      const bool up = (lane & kk) == 0, lower = (lane & jj) == 0;
      v = (lower == up) ? min(v, o) : max(v, o);
    }
}

// bitonic sort of buf[0, M) (M a power of two) by nthr threads, index tid
template <typename SYNC>
__device__ __forceinline__ void bitonic_u32(uint32_t *buf, uint32_t M, uint32_t tid, uint32_t nthr,
                                            SYNC sync) {
  for (uint32_t kk = 2; kk <= M; kk <<= 1)
    for (uint32_t jj = kk >> 1; jj > 0; jj >>= 1) {
      for (uint32_t t = tid; t < (M >> 1); t += nthr) {
        const uint32_t a = ((t & ~(jj - 1)) << 1) | (t & (jj - 1));
        const uint32_t b = (jj == (kk >> 1)) ? (a ^ (kk - 1)) : (a + jj);
        const uint32_t va = buf[a], vb = buf[b];
        if (vb < va) {
          buf[a] = vb;
          buf[b] = va;
        }
      }
      sync();
    }
}

__global__ void __launch_bounds__(kSWT) segsort_warp_kernel(const __grid_constant__ GroupArgs g) {
  __shared__ uint32_t buf[kSWT / 32][kSWBuf];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const unsigned long long n = *g.seg_count;
  const unsigned long long nwarps = (unsigned long long)gridDim.x * (kSWT / 32);
  for (unsigned long long x = (unsigned long long)blockIdx.x * (kSWT / 32) + w; x < n; x += nwarps) {
    const uint32_t m = g.seg_len[x];
    if (m > (uint32_t)kSWBuf) continue;
    uint32_t *p = g.members + g.seg_pos[x];
    if (m <= 32) {
      uint32_t v = (uint32_t)lane < m ? p[lane] : ~0u;
      bitonic32_u32(v, lane);
      if ((uint32_t)lane < m) p[lane] = v;
      continue;
    }
    uint32_t M = 64;
    while (M < m) M <<= 1;
    for (uint32_t i = lane; i < M; i += 32) buf[w][i] = i < m ? p[i] : ~0u;
    __syncwarp();
    bitonic_u32(buf[w], M, lane, 32, [] { __syncwarp(); });
    for (uint32_t i = lane; i < m; i += 32) p[i] = buf[w][i];
    __syncwarp();
  }
}

__global__ void __launch_bounds__(1024) segsort_cta_kernel(const __grid_constant__ GroupArgs g) {
  extern __shared__ uint32_t cbuf[];
  const unsigned long long n = *g.seg_count;
  for (unsigned long long x = blockIdx.x; x < n; x += gridDim.x) {
    const uint32_t m = g.seg_len[x];
    if (m <= (uint32_t)kSWBuf) continue;
    uint32_t *p = g.members + g.seg_pos[x];
    uint32_t M = 1;
    while (M < m) M <<= 1;
    if (M <= (uint32_t)kSCBuf) {
      for (uint32_t i = threadIdx.x; i < M; i += blockDim.x) cbuf[i] = i < m ? p[i] : ~0u;
      __syncthreads();
      bitonic_u32(cbuf, M, threadIdx.x, blockDim.x, [] { __syncthreads(); });
      for (uint32_t i = threadIdx.x; i < m; i += blockDim.x) p[i] = cbuf[i];
      __syncthreads();
    } else {
      // a group of more than 16K generators: in place in global memory
      for (uint32_t kk = 2; kk <= M; kk <<= 1)
        for (uint32_t jj = kk >> 1; jj > 0; jj >>= 1) {
          for (uint32_t t = threadIdx.x; t < (M >> 1); t += blockDim.x) {
            const uint32_t a = ((t & ~(jj - 1)) << 1) | (t & (jj - 1));
            const uint32_t b = (jj == (kk >> 1)) ? (a ^ (kk - 1)) : (a + jj);
            if (b < m) {
              const uint32_t va = p[a], vb = p[b];
              if (vb < va) {
                p[a] = vb;
                p[b] = va;
              }
            }
          }
          __syncthreads();
        }
    }
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
  const int B = a.plan.bits1;
  if (B < 0 || B > kMaxB1) return cudaErrorInvalidValue;
  const int64_t nb = (int64_t)1 << B;
  cudaError_t e = cudaMemsetAsync(a.bsize1, 0, (size_t)(a.plan.c * nb) * 4, st);
  if (e != cudaSuccess || a.plan.nchunks == 0) return e;     // no pairs: every bucket empty
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
  int per_sm = 1;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, scatter_c_kernel, kAT, smem);
  const int grid = (int)std::min<int64_t>((int64_t)num_sms * std::max(per_sm, 1), a.plan.nchunks);
  scatter_c_kernel<<<grid, kAT, smem, st>>>(a);
  ++g_launches;
  return cudaGetLastError();
}

cudaError_t group_c_segsort(const GroupArgs &a, int num_sms, cudaStream_t st) {
  segsort_warp_kernel<<<num_sms * 8, kSWT, 0, st>>>(a);
  ++g_launches;
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return e;
  const size_t smem = (size_t)kSCBuf * 4;
  if ((e = cudaFuncSetAttribute(segsort_cta_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                (int)smem)) != cudaSuccess)
    return e;
  segsort_cta_kernel<<<num_sms, 1024, smem, st>>>(a);
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
