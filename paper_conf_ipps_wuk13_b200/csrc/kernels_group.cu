// kernels_group.cu — grouping of <shingle, generator> pairs into tuples
// <s_j, L(s_j)> "once for each random trial" (AMB-5) for sm_100a.
//
// The paper sorts on the CPU (Alg. 2 l.16); a full LSD radix sort of
// 64-bit keys would move ~200 B/pair through HBM.  Here:
//   1. hist    : per (trial, chunk) histogram of the top B key bits;
//   2. offsets : column prefix over chunks + per-trial bucket scan;
//   3. scatter : one MSD pass into (trial, bucket) order (unstable, smem
//                cursors; 12 B/pair written);
//   4. local   : one CTA per bucket sorts it in shared memory by the total
//                order (key, member) — counting sort on the next 12 key bits,
//                insertion sort of tiny sub-bins, a bitonic network for
//                large ones (runs of equal keys = big groups) — and writes
//                the members plus one head bit per group start (the RLE);
//   5. big     : buckets above the smem capacity, one CTA each, bitonic sort
//                in global (L2-resident) memory.
// Members are unique within a trial (one pair per row and trial), so
// (key, member) is a strict total order: the result is deterministic and
// equal to a stable sort by key of the member-ascending input.
#include <algorithm>

#include "kernels.h"
#include "scan.cuh"
#include "sg_internal.cuh"

namespace sg {

namespace {

constexpr int kGThreads = 512;
constexpr int kLocalCap = 4096;      // elements sorted in smem per bucket
constexpr int kSubBits = 12;
constexpr int kNSub = 1 << kSubBits;
constexpr int kInsertionMax = 16;
constexpr int kMaxLarge = 256;

__device__ __forceinline__ uint32_t bin_of(uint64_t key, int bits) {
  return bits ? (uint32_t)(key >> (64 - bits)) : 0u;
}

__device__ __forceinline__ uint32_t sub_of(uint64_t key, int bits) {
  return (uint32_t)((key << bits) >> (64 - kSubBits));
}

__device__ __forceinline__ bool pair_less(uint64_t ka, uint32_t va, uint64_t kb, uint32_t vb) {
  return ka < kb || (ka == kb && va < vb);
}

__device__ __forceinline__ uint32_t val_at(const GroupArgs &g, int64_t gi, int64_t iseg) {
  if (g.vals) return g.vals[gi];
  if (g.rowid) return g.rowid[iseg];
  return g.val_base + (uint32_t)iseg;
}

// ---- 1. histogram -----------------------------------------------------------
__global__ void __launch_bounds__(kGThreads) hist_kernel(const __grid_constant__ GroupArgs g) {
  extern __shared__ uint32_t hist[];
  const int64_t nb = g.plan.nbins;
  const int bits = g.plan.bits;
  for (int64_t i = threadIdx.x; i < nb; i += blockDim.x) hist[i] = 0;
  __syncthreads();
  const int64_t k = blockIdx.x;
  const int64_t st = g.plan.chunk_start[k];
  const int len = g.plan.chunk_len[k];
  const uint64_t *__restrict__ keys = g.keys + st;
  for (int i = threadIdx.x; i < len; i += blockDim.x) atomicAdd(&hist[bin_of(keys[i], bits)], 1u);
  __syncthreads();
  uint32_t *out = g.counts + k * nb;
  for (int64_t i = threadIdx.x; i < nb; i += blockDim.x) out[i] = hist[i];
}

// ---- 2. offsets ---------------------------------------------------------------
// counts[k][b] <- exclusive prefix over the chunks of its trial; bsize[j][b].
__global__ void colscan_kernel(const __grid_constant__ GroupArgs g) {
  const int64_t nb = g.plan.nbins;
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
  g.bsize[(int64_t)j * nb + b] = run;
}

// bstart[j][b] = exclusive scan of bsize[j][.] (relative to the segment).
__global__ void binscan_kernel(const __grid_constant__ GroupArgs g) {
  __shared__ int64_t ws[33];
  const int64_t nb = g.plan.nbins;
  const int j = blockIdx.x;
  const uint32_t *sz = g.bsize + (int64_t)j * nb;
  uint32_t *out = g.bstart + (int64_t)j * nb;
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

// ---- 3. scatter ---------------------------------------------------------------
__global__ void __launch_bounds__(kGThreads) scatter_kernel(const __grid_constant__ GroupArgs g) {
  extern __shared__ uint32_t cur[];
  const int64_t nb = g.plan.nbins;
  const int bits = g.plan.bits;
  const int64_t k = blockIdx.x;
  const int j = g.plan.chunk_trial[k];
  const uint32_t *pre = g.counts + k * nb;
  const uint32_t *bst = g.bstart + (int64_t)j * nb;
  for (int64_t i = threadIdx.x; i < nb; i += blockDim.x) cur[i] = bst[i] + pre[i];
  __syncthreads();
  const int64_t st = g.plan.chunk_start[k];
  const int64_t seg = g.plan.seg[j];
  const int len = g.plan.chunk_len[k];
  for (int i = threadIdx.x; i < len; i += blockDim.x) {
    const int64_t gi = st + i;
    const uint64_t key = g.keys[gi];
    const uint32_t val = val_at(g, gi, gi - seg);
    const uint32_t pos = atomicAdd(&cur[bin_of(key, bits)], 1u);
    g.bkeys[seg + pos] = key;
    g.bvals[seg + pos] = val;
  }
}

// ---- shared epilogue: members + head bits ------------------------------------
// Sorted order given by idx(p) into (K, V); writes members[gbase + p] and the
// head bit of each p whose key differs from its predecessor's.
template <typename KF, typename VF>
__device__ __forceinline__ void write_groups(const GroupArgs &g, int64_t gbase, int n, KF keyat,
                                             VF valat) {
  for (int p = threadIdx.x; p < n; p += blockDim.x) g.members[gbase + p] = valat(p);
  const int64_t w0 = gbase >> 5, w1 = (gbase + n - 1) >> 5;
  for (int64_t w = w0 + threadIdx.x; w <= w1; w += blockDim.x) {
    uint32_t bits = 0;
    const int64_t lo = max(gbase, w << 5), hi = min(gbase + n, (w << 5) + 32);
    for (int64_t gp = lo; gp < hi; ++gp) {
      const int p = (int)(gp - gbase);
      const bool h = (p == 0) || keyat(p) != keyat(p - 1);
      bits |= (uint32_t)h << (gp & 31);
    }
    if (lo == (w << 5) && hi == (w << 5) + 32) g.head[w] = bits;
    else if (bits) atomicOr(&g.head[w], bits);
  }
}

// ---- 4. local sort ------------------------------------------------------------
struct LocalSmem {
  uint64_t K[kLocalCap];
  uint32_t V[kLocalCap];
  uint16_t perm[kLocalCap];
  uint32_t sub[kNSub];
  int64_t ws[33];
  uint32_t large_st[kMaxLarge];
  uint32_t large_n[kMaxLarge];
  int nlarge;
};

__device__ __forceinline__ void bitonic_perm(LocalSmem &S, int st, int m) {
  int M = 1;
  while (M < m) M <<= 1;
  uint16_t *pm = S.perm + st;
  for (int k = 2; k <= M; k <<= 1) {
    for (int jj = k >> 1; jj > 0; jj >>= 1) {
      for (int t = threadIdx.x; t < (M >> 1); t += blockDim.x) {
        int i, l;
        if (jj == (k >> 1)) {          // flip step: pair i with the mirror in its k-block
          i = (t / jj) * k + (t % jj);
          l = (i / k) * k + (k - 1 - (i % k));
        } else {
          i = (t / jj) * (jj << 1) + (t % jj);
          l = i + jj;
        }
        if (l < m) {
          const int a = pm[i], b = pm[l];
          if (pair_less(S.K[b], S.V[b], S.K[a], S.V[a])) {
            pm[i] = (uint16_t)b;
            pm[l] = (uint16_t)a;
          }
        }
      }
      __syncthreads();
    }
  }
}

__global__ void __launch_bounds__(kGThreads) local_kernel(const __grid_constant__ GroupArgs g) {
  extern __shared__ __align__(16) unsigned char smraw[];
  LocalSmem &S = *reinterpret_cast<LocalSmem *>(smraw);
  const int64_t q = blockIdx.x;
  const int64_t nb = g.plan.nbins;
  const int j = (int)(q / nb);
  const int n = (int)min(g.bsize[q], 0x7FFFFFFFu);
  if (n == 0) return;
  if (n > kLocalCap) {
    if (threadIdx.x == 0) g.big_list[atomicAdd(g.big_count, 1u)] = (uint32_t)q;
    return;
  }
  const int bits = g.plan.bits;
  const int64_t gbase = g.plan.seg[j] + g.bstart[q];
  for (int i = threadIdx.x; i < n; i += blockDim.x) {
    S.K[i] = g.bkeys[gbase + i];
    S.V[i] = g.bvals[gbase + i];
  }
  for (int i = threadIdx.x; i < kNSub; i += blockDim.x) S.sub[i] = 0;
  if (threadIdx.x == 0) S.nlarge = 0;
  __syncthreads();
  for (int i = threadIdx.x; i < n; i += blockDim.x) atomicAdd(&S.sub[sub_of(S.K[i], bits)], 1u);
  __syncthreads();
  {
    constexpr int per = kNSub / kGThreads;
    uint32_t v[per];
    int64_t sum = 0;
#pragma unroll
    for (int k = 0; k < per; ++k) {
      v[k] = S.sub[threadIdx.x * per + k];
      sum += v[k];
    }
    int64_t tot;
    int64_t ex = block_excl_scan<int64_t>(sum, S.ws, &tot);
#pragma unroll
    for (int k = 0; k < per; ++k) {
      S.sub[threadIdx.x * per + k] = (uint32_t)ex;
      ex += v[k];
    }
  }
  __syncthreads();
  for (int i = threadIdx.x; i < n; i += blockDim.x)
    S.perm[atomicAdd(&S.sub[sub_of(S.K[i], bits)], 1u)] = (uint16_t)i;
  __syncthreads();
  // S.sub[d] is now the end of sub-bin d
  for (int d = threadIdx.x; d < kNSub; d += blockDim.x) {
    const int st = d ? (int)S.sub[d - 1] : 0;
    const int m = (int)S.sub[d] - st;
    if (m < 2) continue;
    if (m <= kInsertionMax) {
      uint16_t *pm = S.perm + st;
      for (int x = 1; x < m; ++x) {
        const uint16_t e = pm[x];
        const uint64_t ke = S.K[e];
        const uint32_t ve = S.V[e];
        int y = x - 1;
        while (y >= 0 && pair_less(ke, ve, S.K[pm[y]], S.V[pm[y]])) {
          pm[y + 1] = pm[y];
          --y;
        }
        pm[y + 1] = e;
      }
    } else {
      int slot = atomicAdd(&S.nlarge, 1);
      if (slot < kMaxLarge) {
        S.large_st[slot] = st;
        S.large_n[slot] = m;
      }
    }
  }
  __syncthreads();
  const int nl = S.nlarge;
  if (nl > kMaxLarge) {
    // pathological: too many large sub-bins; sort the whole bucket
    bitonic_perm(S, 0, n);
  } else {
    for (int x = 0; x < nl; ++x) bitonic_perm(S, S.large_st[x], S.large_n[x]);
  }
  __syncthreads();
  write_groups(g, gbase, n, [&](int p) { return S.K[S.perm[p]]; },
               [&](int p) { return S.V[S.perm[p]]; });
}

// ---- 5. big buckets (global-memory bitonic, one CTA each) ----------------------
__global__ void __launch_bounds__(1024) big_kernel(const __grid_constant__ GroupArgs g) {
  const int64_t q = g.big_list[blockIdx.x];
  const int64_t nb = g.plan.nbins;
  const int j = (int)(q / nb);
  const int64_t n = g.bsize[q];
  const int64_t gbase = g.plan.seg[j] + g.bstart[q];
  uint64_t *K = g.bkeys + gbase;
  uint32_t *V = g.bvals + gbase;
  int64_t M = 1;
  while (M < n) M <<= 1;
  for (int64_t k = 2; k <= M; k <<= 1) {
    for (int64_t jj = k >> 1; jj > 0; jj >>= 1) {
      for (int64_t t = threadIdx.x; t < (M >> 1); t += blockDim.x) {
        int64_t i, l;
        if (jj == (k >> 1)) {
          i = (t / jj) * k + (t % jj);
          l = (i / k) * k + (k - 1 - (i % k));
        } else {
          i = (t / jj) * (jj << 1) + (t % jj);
          l = i + jj;
        }
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
  // members + head bits (n may exceed int range only for absurd inputs)
  for (int64_t p = threadIdx.x; p < n; p += blockDim.x) g.members[gbase + p] = V[p];
  const int64_t w0 = gbase >> 5, w1 = (gbase + n - 1) >> 5;
  for (int64_t w = w0 + threadIdx.x; w <= w1; w += blockDim.x) {
    uint32_t bits = 0;
    const int64_t lo = max(gbase, w << 5), hi = min(gbase + n, (w << 5) + 32);
    for (int64_t gp = lo; gp < hi; ++gp) {
      const int64_t p = gp - gbase;
      const bool h = (p == 0) || K[p] != K[p - 1];
      bits |= (uint32_t)h << (gp & 31);
    }
    if (lo == (w << 5) && hi == (w << 5) + 32) g.head[w] = bits;
    else if (bits) atomicOr(&g.head[w], bits);
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

__global__ void transpose_ids_kernel(const uint64_t *__restrict__ keys, int64_t nrows, int c,
                                     uint64_t *ids) {
  const int64_t tot = nrows * c;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < tot;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = i / c, j = i % c;
    ids[i] = fmix_inv(keys[j * nrows + r]);
  }
}

}  // namespace

int64_t group_local_capacity() { return kLocalCap; }

cudaError_t group_hist(const GroupArgs &g, cudaStream_t st) {
  if (g.plan.nchunks == 0) return cudaSuccess;
  size_t smem = (size_t)g.plan.nbins * sizeof(uint32_t);
  cudaError_t e = cudaFuncSetAttribute(hist_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       (int)smem);
  if (e != cudaSuccess) return e;
  hist_kernel<<<(unsigned)g.plan.nchunks, kGThreads, smem, st>>>(g);
  ++g_launches;
  return cudaGetLastError();
}

cudaError_t group_offsets(const GroupArgs &g, cudaStream_t st) {
  dim3 grid((unsigned)((g.plan.nbins + 255) / 256), (unsigned)g.plan.c);
  colscan_kernel<<<grid, 256, 0, st>>>(g);
  ++g_launches;
  binscan_kernel<<<(unsigned)g.plan.c, 1024, 0, st>>>(g);
  ++g_launches;
  return cudaGetLastError();
}

cudaError_t group_scatter(const GroupArgs &g, cudaStream_t st) {
  if (g.plan.nchunks == 0) return cudaSuccess;
  size_t smem = (size_t)g.plan.nbins * sizeof(uint32_t);
  cudaError_t e = cudaFuncSetAttribute(scatter_kernel,
                                       cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  scatter_kernel<<<(unsigned)g.plan.nchunks, kGThreads, smem, st>>>(g);
  ++g_launches;
  return cudaGetLastError();
}

cudaError_t group_local(const GroupArgs &g, cudaStream_t st) {
  int64_t nq = (int64_t)g.plan.c * g.plan.nbins;
  if (nq == 0) return cudaSuccess;
  size_t smem = sizeof(LocalSmem);
  cudaError_t e = cudaFuncSetAttribute(local_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       (int)smem);
  if (e != cudaSuccess) return e;
  local_kernel<<<(unsigned)nq, kGThreads, smem, st>>>(g);
  ++g_launches;
  return cudaGetLastError();
}

cudaError_t group_big(const GroupArgs &g, uint32_t nbig, cudaStream_t st) {
  if (nbig == 0) return cudaSuccess;
  big_kernel<<<nbig, 1024, 0, st>>>(g);
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
  ++g_launches;
  return cudaGetLastError();
}

cudaError_t sum_i32(const int32_t *a, int64_t n, unsigned long long *d_out, cudaStream_t st) {
  cudaError_t e = cudaMemsetAsync(d_out, 0, sizeof(unsigned long long), st);
  if (e != cudaSuccess || n == 0) return e;
  int grid = (int)std::min<int64_t>((n + 255) / 256, 148 * 8);
  sum_i32_kernel<<<grid, 256, 0, st>>>(a, n, d_out);
  return cudaGetLastError();
}

cudaError_t transpose_keys_to_ids(const uint64_t *keys, int64_t nrows, int32_t c, uint64_t *ids,
                                  cudaStream_t st) {
  int64_t tot = nrows * c;
  if (tot == 0) return cudaSuccess;
  int grid = (int)std::min<int64_t>((tot + 255) / 256, 148 * 16);
  transpose_ids_kernel<<<grid, 256, 0, st>>>(keys, nrows, c, ids);
  ++g_launches;
  return cudaGetLastError();
}

}  // namespace sg
