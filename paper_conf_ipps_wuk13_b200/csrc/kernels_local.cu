// kernels_local.cu — sort inside one key bucket and run-length segmentation:
// the second half of the per-trial grouping (AMB-5).
//
// local_kernel: persistent, one CTA (1024 threads) per SM, buckets of up to
// 8192 pairs double-buffered into shared memory with cp.async.  Per bucket:
//   * counting sort on the next <= 11 key bits (sub-bins of ~1-2 pairs);
//   * element-parallel placement: every pair counts the pairs of its sub-bin
//     that precede it in (key, member) order -> its position; it opens a group
//     (head bit) iff no pair with an equal key has a smaller member;
//   * sub-bins with > 64 pairs (long runs of one key = big groups) are
//     bitonic-sorted by a warp (<= 256) or by the whole CTA;
//   * members are written at bucket offset + position, the head bits as
//     32-bit words (atomicOr on the two words shared with neighbours).
// big_kernel: buckets above 8192 pairs, one CTA each, bitonic sort in global
// (L2-resident) memory.
#include <algorithm>

#include "group_common.cuh"
#include "kernels.h"
#include "scan.cuh"
#include "sg_internal.cuh"

namespace sg {

namespace {

using grp::bitonic_idx;
using grp::bucket_extent;
using grp::pair_less;

constexpr int kLocalCap = 8192;
constexpr int kLThreads = 1024;
constexpr int kMaxSubBits = 11;
constexpr int kNSubMax = 1 << kMaxSubBits;
constexpr int kRankMax = 64;         // sub-bins up to this size: element-parallel ranks
constexpr int kWarpSortMax = 256;    // then warp bitonic, then CTA bitonic
constexpr int kMaxList = 64;

struct LocalSmem {
  uint64_t K[2][kLocalCap];
  uint32_t V[2][kLocalCap];
  uint16_t perm[kLocalCap];
  uint32_t sub[kNSubMax];
  uint32_t hb[kLocalCap / 32 + 2];
  int64_t ws[33];
  uint32_t run_st[kMaxList];
  uint32_t run_n[kMaxList];
  int nrun;
};

__device__ __forceinline__ void cp_async8(void *sdst, const void *gsrc) {
  const unsigned s = (unsigned)__cvta_generic_to_shared(sdst);
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8;\n" ::"r"(s), "l"(gsrc));
}
__device__ __forceinline__ void cp_async4(void *sdst, const void *gsrc) {
  const unsigned s = (unsigned)__cvta_generic_to_shared(sdst);
  asm volatile("cp.async.ca.shared.global [%0], [%1], 4;\n" ::"r"(s), "l"(gsrc));
}
__device__ __forceinline__ void cp_commit() { asm volatile("cp.async.commit_group;\n" ::); }
__device__ __forceinline__ void cp_wait1() { asm volatile("cp.async.wait_group 1;\n" ::); }

__device__ __forceinline__ void prefetch_bucket(LocalSmem &S, int buf, const GroupArgs &g,
                                                int64_t sbase, int64_t n) {
  if (n > kLocalCap) n = 0;
  for (int i = threadIdx.x; i < n; i += blockDim.x) {
    cp_async8(&S.K[buf][i], g.bkeys + sbase + i);
    cp_async4(&S.V[buf][i], g.bvals + sbase + i);
  }
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

__global__ void __launch_bounds__(kLThreads, 1) local_kernel(const __grid_constant__ GroupArgs g) {
  extern __shared__ __align__(16) unsigned char smraw[];
  LocalSmem &S = *reinterpret_cast<LocalSmem *>(smraw);
  const int64_t nq = (int64_t)g.plan.c * g.plan.nbins;
  const int bits = g.plan.bits;
  const int64_t obase = g.plan.seg[0];     // scratch -> output position
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5, nwarp = blockDim.x >> 5;
  int64_t q = blockIdx.x;
  int cur = 0;
  int64_t sb = 0, n64 = 0;
  if (q < nq) {
    bucket_extent(g, q, sb, n64);
    prefetch_bucket(S, 0, g, sb, n64);
  }
  cp_commit();
  for (; q < nq; q += gridDim.x) {
    const int64_t qn = q + gridDim.x;
    int64_t sbn = 0, nn = 0;
    if (qn < nq) {
      bucket_extent(g, qn, sbn, nn);
      prefetch_bucket(S, cur ^ 1, g, sbn, nn);
    }
    cp_commit();
    cp_wait1();
    __syncthreads();
    if (n64 > kLocalCap) {
      if (threadIdx.x == 0) g.big_list[atomicAdd(g.big_count, 1u)] = (uint32_t)q;
    } else if (n64 > 0) {
      const int n = (int)n64;
      const uint64_t *K = S.K[cur];
      const uint32_t *V = S.V[cur];
      int sbits = 1;
      while ((1 << sbits) < n && sbits < kMaxSubBits) ++sbits;
      const int nsub = 1 << sbits;
      const int nhw = (n + 31) >> 5;
      for (int i = threadIdx.x; i < nsub; i += blockDim.x) S.sub[i] = 0;
      for (int i = threadIdx.x; i < nhw; i += blockDim.x) S.hb[i] = 0;
      if (threadIdx.x == 0) S.nrun = 0;
      __syncthreads();
      auto subof = [&](uint64_t key) { return (uint32_t)((key << bits) >> (64 - sbits)); };
      for (int i = threadIdx.x; i < n; i += blockDim.x) atomicAdd(&S.sub[subof(K[i])], 1u);
      __syncthreads();
      {
        const int per = (nsub + blockDim.x - 1) / blockDim.x;   // <= 2
        const int b0 = threadIdx.x * per;
        uint32_t v0 = (per > 0 && b0 < nsub) ? S.sub[b0] : 0u;
        uint32_t v1 = (per > 1 && b0 + 1 < nsub) ? S.sub[b0 + 1] : 0u;
        int64_t tot;
        const int64_t ex = block_excl_scan<int64_t>((int64_t)v0 + v1, S.ws, &tot);
        if (per > 0 && b0 < nsub) S.sub[b0] = (uint32_t)ex;
        if (per > 1 && b0 + 1 < nsub) S.sub[b0 + 1] = (uint32_t)(ex + v0);
      }
      __syncthreads();
      for (int i = threadIdx.x; i < n; i += blockDim.x)
        S.perm[atomicAdd(&S.sub[subof(K[i])], 1u)] = (uint16_t)i;
      __syncthreads();
      // S.sub[d] is now the end of sub-bin d; element-parallel placement
      const int64_t gbase = obase + sb;
      for (int i = threadIdx.x; i < n; i += blockDim.x) {
        const uint64_t ki = K[i];
        const uint32_t vi = V[i];
        const uint32_t d = subof(ki);
        const int en = (int)S.sub[d];
        const int st = d ? (int)S.sub[d - 1] : 0;
        const int m = en - st;
        int pos, eq = 0;
        if (m == 1) {
          pos = st;
        } else if (m <= kRankMax) {
          int rank = 0;
          for (int x = st; x < en; ++x) {
            const int e = S.perm[x];
            const uint64_t ke = K[e];
            const uint32_t ve = V[e];
            rank += pair_less(ke, ve, ki, vi);
            eq += (ke == ki) & (ve < vi);
          }
          pos = st + rank;
        } else {
          if (S.perm[st] == i) {                   // one representative registers the run
            const int s = atomicAdd(&S.nrun, 1);
            if (s < kMaxList) {
              S.run_st[s] = st;
              S.run_n[s] = m;
            }
          }
          continue;
        }
        g.members[gbase + pos] = vi;
        if (eq == 0) atomicOr(&S.hb[pos >> 5], 1u << (pos & 31));
      }
      __syncthreads();
      const int nrun = S.nrun;
      if (nrun > 0) {
        if (nrun > kMaxList) {
          // more long runs than list slots: sort the whole bucket and place it
          bitonic_idx(S.perm, n, K, V, threadIdx.x, blockDim.x, [] { __syncthreads(); });
          for (int i = threadIdx.x; i < nhw; i += blockDim.x) S.hb[i] = 0;
          __syncthreads();
          for (int p = threadIdx.x; p < n; p += blockDim.x) {
            const int e = S.perm[p];
            g.members[gbase + p] = V[e];
            if (p == 0 || K[S.perm[p - 1]] != K[e]) atomicOr(&S.hb[p >> 5], 1u << (p & 31));
          }
        } else {
          for (int x = wid; x < nrun; x += nwarp) {
            if (S.run_n[x] <= kWarpSortMax)
              bitonic_idx(S.perm + S.run_st[x], (int)S.run_n[x], K, V, lane, 32, [] { __syncwarp(); });
          }
          for (int x = 0; x < nrun; ++x) {
            if (S.run_n[x] > kWarpSortMax)
              bitonic_idx(S.perm + S.run_st[x], (int)S.run_n[x], K, V, threadIdx.x, blockDim.x,
                          [] { __syncthreads(); });
          }
          __syncthreads();
          for (int x = 0; x < nrun; ++x) {
            const int st = (int)S.run_st[x], m = (int)S.run_n[x];
            for (int t = threadIdx.x; t < m; t += blockDim.x) {
              const int p = st + t;
              const int e = S.perm[p];
              g.members[gbase + p] = V[e];
              if (t == 0 || K[S.perm[p - 1]] != K[e]) atomicOr(&S.hb[p >> 5], 1u << (p & 31));
            }
          }
        }
        __syncthreads();
      }
      store_heads(g.head, S.hb, gbase, n);
    }
    __syncthreads();
    cur ^= 1;
    sb = sbn;
    n64 = nn;
  }
  asm volatile("cp.async.wait_all;\n" ::);
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
  for (int64_t p = threadIdx.x; p < n; p += blockDim.x) g.members[gbase + p] = V[p];
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
  const int grid = (int)std::min<int64_t>((int64_t)num_sms, nq);
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
