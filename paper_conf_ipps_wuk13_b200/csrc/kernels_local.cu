// kernels_local.cu — sort inside one key bucket and run-length segmentation:
// the second half of the per-trial grouping (AMB-5).
//
// The partition (kernels_group.cu) is stable, so inside a bucket the pairs
// of one trial are still in generator order and a STABLE sort by key alone
// yields the canonical (key, member) order.
//
// local_kernel: persistent CTAs of 8 warps (3 per SM overlap each other's
// loads), one bucket of up to 4096 pairs at a time in shared memory:
//   * two stable LSD multi-split passes on the 16 key bits after the bucket
//     bits (8 bits each; warp segments, __match_any_sync ranks, a bin-major
//     [digit][warp] counter matrix turned into starts by one block scan): the
//     pairs of one group stay together and in member order;
//   * the rare runs where distinct keys share those 16 bits out of order get
//     a stable insertion sort by key;
//   * members are written in sorted order (coalesced), one head bit per group
//     start (ballot per 32 positions).
// big_kernel: buckets above 4096 pairs, one CTA each, bitonic sort by the
// total order (key, member) in global (L2-resident) memory.
#include <algorithm>

#include "group_common.cuh"
#include "kernels.h"
#include "scan.cuh"
#include "sg_internal.cuh"

namespace sg {

namespace {

using grp::bucket_extent;
using grp::pair_less;

constexpr int kLocalCap = 4096;
constexpr int kLThreads = 256;
constexpr int kLWarps = kLThreads / 32;
constexpr int kPerLane = kLocalCap / kLThreads;   // 16
constexpr int kDigitBits = 8;                     // two stable LSD passes = 16 key bits
constexpr int kDigits = 1 << kDigitBits;
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

__device__ __forceinline__ uint32_t lanemask_lt() {
  uint32_t m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}

// One stable multi-split pass over n <= 4096 elements: warp w owns the
// positions [w*seg, (w+1)*seg) of the current order src (identity if null)
// and writes the new order to dst, stable on digit(key).
template <typename DIG>
__device__ __forceinline__ void lsd_pass(LocalSmem &S, int n, const uint16_t *src, uint16_t *dst,
                                         DIG digit) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const uint32_t lt = lanemask_lt();
  const int seg = (n + kLWarps - 1) / kLWarps;     // <= 512
  reinterpret_cast<uint4 *>(S.cnt)[threadIdx.x] = make_uint4(0, 0, 0, 0);
  __syncthreads();
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
  }
  __syncthreads();
}

// Head-bit words of output positions [gbase, gbase + n) from the bucket-local
// bit array hb (bit p = position p).
__device__ __forceinline__ void store_heads(uint32_t *head, const uint32_t *hb, int64_t gbase,
                                            int n) {
  const int64_t w0 = gbase >> 5, w1 = (gbase + n - 1) >> 5;
  const int off = (int)(gbase & 31);
  const int nw = (n + 31) >> 5;
  for (int64_t w = w0 + threadIdx.x; w <= w1; w += blockDim.x) {
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

__global__ void __launch_bounds__(kLThreads, 2) local_kernel(const __grid_constant__ GroupArgs g) {
  extern __shared__ __align__(16) unsigned char smraw[];
  LocalSmem &S = *reinterpret_cast<LocalSmem *>(smraw);
  const int64_t nq = (int64_t)g.plan.c * g.plan.nbins;
  const int bits = g.plan.bits;
  const int64_t obase = g.plan.seg[0];     // scratch -> output position
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  for (int64_t q = blockIdx.x; q < nq; q += gridDim.x) {
    int64_t sb, n64;
    bucket_extent(g, q, sb, n64);
    if (n64 == 0) continue;
    if (n64 > kLocalCap) {
      if (threadIdx.x == 0) g.big_list[atomicAdd(g.big_count, 1u)] = (uint32_t)q;
      continue;
    }
    const int n = (int)n64;
    for (int i = threadIdx.x; i < n; i += kLThreads) {
      const unsigned sk = (unsigned)__cvta_generic_to_shared(&S.K[i]);
      const unsigned sv = (unsigned)__cvta_generic_to_shared(&S.V[i]);
      asm volatile("cp.async.ca.shared.global [%0], [%1], 8;\n" ::"r"(sk), "l"(g.bkeys + sb + i));
      asm volatile("cp.async.ca.shared.global [%0], [%1], 4;\n" ::"r"(sv), "l"(g.bvals + sb + i));
    }
    asm volatile("cp.async.commit_group;\ncp.async.wait_all;\n" ::);
    // (lsd_pass begins with a barrier after zeroing its counters)
    lsd_pass(S, n, nullptr, S.perm[0],
             [&](uint64_t key) { return (uint32_t)((key << (bits + 8)) >> 56); });
    lsd_pass(S, n, S.perm[0], S.perm[1],
             [&](uint64_t key) { return (uint32_t)((key << bits) >> 56); });
    const uint16_t *pm = S.perm[1];
    const uint64_t *K = S.K;
    auto d16 = [&](uint64_t key) { return (uint32_t)((key << bits) >> 48); };
    // ---- rare: distinct keys sharing the 16 bits out of key order -> a
    // stable insertion sort of that run (registered once via its start bit)
    for (int i = threadIdx.x; i < (kLocalCap / 32 + 2); i += blockDim.x) S.hb[i] = 0;
    if (threadIdx.x == 0) S.nfix = 0;
    __syncthreads();
    for (int p = threadIdx.x + 1; p < n; p += blockDim.x) {
      const uint64_t kp = K[pm[p]];
      if (kp < K[pm[p - 1]]) {
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
          int y = x - 1;
          while (y >= 0 && ke < K[q2[y]]) { q2[y + 1] = q2[y]; --y; }
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
        int y = x - 1;
        while (y >= a && ke < K[q2[y]]) { q2[y + 1] = q2[y]; --y; }   // strict: stable
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
    store_heads(g.head, S.hb, gbase, n);
    __syncthreads();
  }
}

// ---- big buckets: one CTA, bitonic in global memory ---------------------------
__global__ void __launch_bounds__(1024) big_kernel(const __grid_constant__ GroupArgs g) {
  const int64_t q = g.big_list[blockIdx.x];
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
}

}  // namespace

int64_t group_local_capacity() { return kLocalCap; }

cudaError_t group_local(const GroupArgs &g, int num_sms, cudaStream_t st) {
  const int64_t nq = (int64_t)g.plan.c * g.plan.nbins;
  if (nq == 0) return cudaSuccess;
  const size_t smem = sizeof(LocalSmem);
  cudaError_t e = cudaFuncSetAttribute(local_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       (int)smem);
  if (e != cudaSuccess) return e;
  int per_sm = 0;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, local_kernel, kLThreads, smem);
  if (e != cudaSuccess) return e;
  per_sm = std::max(per_sm, 1);
  const int grid = (int)std::min<int64_t>((int64_t)num_sms * per_sm, nq);
  local_kernel<<<grid, kLThreads, smem, st>>>(g);
  ++g_launches;
  return cudaGetLastError();
}

cudaError_t group_big(const GroupArgs &g, uint32_t nbig, cudaStream_t st) {
  if (nbig == 0) return cudaSuccess;
  big_kernel<<<nbig, 1024, 0, st>>>(g);
  ++g_launches;
  return cudaGetLastError();
}

}  // namespace sg
