// kernels_group.cu — partition of <shingle, generator> pairs into per-trial
// key buckets, the first half of the grouping "once for each random trial"
// (AMB-5).  The second half (sort inside a bucket + RLE) is
// kernels_local.cu.  DESIGN.md §6.2.
//
//   1. hist     : per (trial, chunk) histogram of the top bits1 key bits;
//   2. offsets  : column prefix over chunks + per-trial bucket scan;
//   3. scatter  : one persistent CTA per SM writes (key, member) into coarse
//                 (trial, bucket) order through shared-memory cursors.  The
//                 fan-out is <= 1024 buckets, so the partially written
//                 sectors all CTAs keep open (SMs x 1024 x 2 x 32 B < 10 MB)
//                 stay in L2 and every sector reaches HBM complete;
//   4. scatter2 : only when a trial segment is too long for 1024 buckets of
//                 <= 8K pairs: one CTA per coarse bucket histograms it (the
//                 re-read hits L2) and scatters it by the next key bits
//                 (fan-out <= 64) into the final buckets.
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
constexpr int kSThreads = 1024;      // scatter: one persistent CTA per SM
constexpr int kItems = 8;            // ILP batch per thread
constexpr int kMaxSingleBits = 10;   // single-level fan-out bound
constexpr int kCoarseBits = 9;       // two-level: first fan-out
constexpr int kMaxBits = 14;         // final buckets per trial <= 16384

__device__ __forceinline__ uint32_t val_at(const GroupArgs &g, int64_t in_idx, int64_t i) {
  if (g.vals) return g.vals[in_idx];
  if (g.rowid) return g.rowid[i];
  return g.val_base + (uint32_t)i;
}

// ---- 1. histogram -----------------------------------------------------------
__global__ void __launch_bounds__(kGThreads) hist_kernel(const __grid_constant__ GroupArgs g) {
  extern __shared__ uint32_t hist[];
  const int64_t nb = g.plan.nb1;
  const int bits = g.plan.bits1;
  for (int64_t i = threadIdx.x; i < nb; i += blockDim.x) hist[i] = 0;
  __syncthreads();
  const int64_t k = blockIdx.x;
  const int j = g.plan.chunk_trial[k];
  const uint64_t *__restrict__ keys = g.keys + g.plan.in_base[j] + g.plan.chunk_i0[k];
  const int len = g.plan.chunk_len[k];
  for (int base = threadIdx.x; base < len; base += blockDim.x * kItems) {
    uint64_t kk[kItems];
#pragma unroll
    for (int u = 0; u < kItems; ++u) {
      const int i = base + u * blockDim.x;
      kk[u] = i < len ? keys[i] : 0;
    }
#pragma unroll
    for (int u = 0; u < kItems; ++u)
      if (base + u * (int)blockDim.x < len) atomicAdd(&hist[top_bits(kk[u], bits)], 1u);
  }
  __syncthreads();
  uint32_t *out = g.counts + k * nb;
  for (int64_t i = threadIdx.x; i < nb; i += blockDim.x) out[i] = hist[i];
}

// ---- 2. offsets ---------------------------------------------------------------
// counts[k][b] <- exclusive prefix over the chunks of its trial; bsize1[j][b].
__global__ void colscan_kernel(const __grid_constant__ GroupArgs g) {
  const int64_t nb = g.plan.nb1;
  const int j = blockIdx.y;
  const int64_t b = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (b >= nb) return;
  const int k0 = g.plan.trial_chunk0[j], k1 = g.plan.trial_chunk0[j + 1];
  uint32_t run = 0;
  for (int k = k0; k < k1; ++k) {
    uint32_t *p = g.counts + (int64_t)k * nb + b;
    uint32_t v = *p;
    *p = run;
    run += v;
  }
  g.bsize1[(int64_t)j * nb + b] = run;
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

// ---- 3. coarse scatter (persistent) -------------------------------------------
__global__ void __launch_bounds__(kSThreads, 1) scatter_kernel(const __grid_constant__ GroupArgs g) {
  extern __shared__ uint32_t cur[];
  const int64_t nb = g.plan.nb1;
  const int bits = g.plan.bits1;
  for (int64_t k = blockIdx.x; k < g.plan.nchunks; k += gridDim.x) {
    const int j = g.plan.chunk_trial[k];
    const uint32_t *pre = g.counts + k * nb;
    const uint32_t *bst = g.bstart1 + (int64_t)j * nb;
    __syncthreads();
    for (int64_t i = threadIdx.x; i < nb; i += blockDim.x) cur[i] = bst[i] + pre[i];
    __syncthreads();
    const int64_t i0 = g.plan.chunk_i0[k];
    const int64_t in0 = g.plan.in_base[j] + i0;
    const int64_t sseg = g.plan.seg[j] - g.plan.seg[0];   // scratch segment start
    const int len = g.plan.chunk_len[k];
    for (int base = threadIdx.x; base < len; base += blockDim.x * kItems) {
      uint64_t kk[kItems];
      uint32_t vv[kItems];
#pragma unroll
      for (int u = 0; u < kItems; ++u) {
        const int i = base + u * blockDim.x;
        if (i < len) {
          kk[u] = g.keys[in0 + i];
          vv[u] = val_at(g, in0 + i, i0 + i);
        }
      }
#pragma unroll
      for (int u = 0; u < kItems; ++u) {
        const int i = base + u * blockDim.x;
        if (i < len) {
          const uint32_t pos = atomicAdd(&cur[top_bits(kk[u], bits)], 1u);
          g.akeys[sseg + pos] = kk[u];
          g.avals[sseg + pos] = vv[u];
        }
      }
    }
  }
}

// ---- 4. second-level scatter (one CTA per coarse bucket) ----------------------
__global__ void __launch_bounds__(kGThreads, 2) scatter2_kernel(const __grid_constant__ GroupArgs g) {
  __shared__ uint32_t cnt[1 << (kMaxBits - kCoarseBits)];
  __shared__ int64_t ws[33];
  const int64_t q1 = blockIdx.x;                 // (trial, coarse bucket)
  const int64_t nb1 = g.plan.nb1;
  const int j = (int)(q1 / nb1);
  const int b1 = (int)(q1 % nb1);
  const int bits = g.plan.bits, bits2 = g.plan.bits - g.plan.bits1;
  const int nb2 = 1 << bits2;
  const uint32_t mask2 = (uint32_t)nb2 - 1u;
  const int64_t sseg = g.plan.seg[j] - g.plan.seg[0];
  const uint32_t st1 = g.bstart1[q1];
  const int64_t n = g.bsize1[q1];
  const uint64_t *__restrict__ K = g.akeys + sseg + st1;
  const uint32_t *__restrict__ V = g.avals + sseg + st1;
  for (int i = threadIdx.x; i < nb2; i += blockDim.x) cnt[i] = 0;
  __syncthreads();
  for (int64_t base = threadIdx.x; base < n; base += (int64_t)blockDim.x * kItems) {
    uint64_t kk[kItems];
#pragma unroll
    for (int u = 0; u < kItems; ++u) {
      const int64_t i = base + u * blockDim.x;
      kk[u] = i < n ? K[i] : 0;
    }
#pragma unroll
    for (int u = 0; u < kItems; ++u)
      if (base + u * (int64_t)blockDim.x < n) atomicAdd(&cnt[top_bits(kk[u], bits) & mask2], 1u);
  }
  __syncthreads();
  // final bucket starts / sizes of this coarse bucket's sub-buckets
  {
    const int d = threadIdx.x;
    const int64_t v = d < nb2 ? cnt[d] : 0;
    int64_t tot;
    const int64_t ex = block_excl_scan<int64_t>(v, ws, &tot);
    if (d < nb2) {
      const int64_t qf = (int64_t)j * g.plan.nbins + ((int64_t)b1 << bits2) + d;
      g.bstart[qf] = st1 + (uint32_t)ex;
      g.bsize[qf] = (uint32_t)v;
      cnt[d] = st1 + (uint32_t)ex;
    }
  }
  __syncthreads();
  for (int64_t base = threadIdx.x; base < n; base += (int64_t)blockDim.x * kItems) {
    uint64_t kk[kItems];
    uint32_t vv[kItems];
#pragma unroll
    for (int u = 0; u < kItems; ++u) {
      const int64_t i = base + u * blockDim.x;
      if (i < n) {
        kk[u] = K[i];
        vv[u] = V[i];
      }
    }
#pragma unroll
    for (int u = 0; u < kItems; ++u) {
      if (base + u * (int64_t)blockDim.x < n) {
        const uint32_t pos = atomicAdd(&cnt[top_bits(kk[u], bits) & mask2], 1u);
        g.bkeys[sseg + pos] = kk[u];
        g.bvals[sseg + pos] = vv[u];
      }
    }
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

void group_bits(int64_t maxseg, int32_t *bits, int32_t *bits1) {
  // final buckets of <= ~4K pairs on average (the shared-memory sort holds 8K)
  // test hook SG_GROUP_TARGET: smaller target buckets (forces the two-level
  // partition and the big-bucket path on graphs the oracle can check)
  const char *e = getenv("SG_GROUP_TARGET");
  int64_t target = e ? atoll(e) : 4096;
  if (target <= 0) target = 4096;
  int b = 0;
  while ((maxseg >> b) > target && b < kMaxBits) ++b;
  *bits = b;
  *bits1 = b <= kMaxSingleBits ? b : kCoarseBits;
}

cudaError_t group_hist(const GroupArgs &g, cudaStream_t st) {
  if (g.plan.nchunks == 0) return cudaSuccess;
  const size_t smem = (size_t)g.plan.nb1 * sizeof(uint32_t);
  hist_kernel<<<(unsigned)g.plan.nchunks, kGThreads, smem, st>>>(g);
  ++g_launches;
  return cudaGetLastError();
}

cudaError_t group_offsets(const GroupArgs &g, cudaStream_t st) {
  dim3 grid((unsigned)((g.plan.nb1 + 255) / 256), (unsigned)g.plan.c);
  colscan_kernel<<<grid, 256, 0, st>>>(g);
  ++g_launches;
  binscan_kernel<<<(unsigned)g.plan.c, 1024, 0, st>>>(g);
  ++g_launches;
  return cudaGetLastError();
}

cudaError_t group_scatter(const GroupArgs &g, int num_sms, cudaStream_t st) {
  if (g.plan.nchunks == 0) return cudaSuccess;
  const size_t smem = (size_t)g.plan.nb1 * sizeof(uint32_t);
  const int grid = (int)std::min<int64_t>(num_sms, g.plan.nchunks);
  scatter_kernel<<<grid, kSThreads, smem, st>>>(g);
  ++g_launches;
  return cudaGetLastError();
}

cudaError_t group_scatter2(const GroupArgs &g, cudaStream_t st) {
  const int64_t nq1 = (int64_t)g.plan.c * g.plan.nb1;
  if (nq1 == 0 || g.plan.bits == g.plan.bits1) return cudaSuccess;
  scatter2_kernel<<<(unsigned)nq1, kGThreads, 0, st>>>(g);
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
