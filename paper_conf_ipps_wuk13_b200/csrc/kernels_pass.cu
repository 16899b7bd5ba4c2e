// kernels_pass.cu — row selection for a shingling pass: pass I takes every
// vertex with at least s links; pass II takes every first-level
// shingle whose generator list has at least s members (S1').
#include <algorithm>

#include "kernels.h"
#include "scan.cuh"
#include "sg_internal.cuh"

namespace sg {

std::atomic<long long> g_launches{0};

namespace {

constexpr int kSelThreads = 256;
constexpr int kSelItems = 4;
constexpr int kSelPerBlock = kSelThreads * kSelItems;

__global__ void scan_inplace_kernel(int64_t *a, int64_t n, int64_t *total) {
  __shared__ int64_t ws[33];
  int64_t carry = 0;
  for (int64_t base = 0; base < n; base += blockDim.x) {
    int64_t i = base + threadIdx.x;
    int64_t v = i < n ? a[i] : 0;
    int64_t tot;
    int64_t ex = block_excl_scan<int64_t>(v, ws, &tot);
    if (i < n) a[i] = carry + ex;
    carry += tot;
  }
  if (threadIdx.x == 0) {
    a[n] = carry;
    if (total) *total = carry;
  }
}

// ---- pass I selection: deg >= s --------------------------------------------
__global__ void sel_csr_count_kernel(const int64_t *__restrict__ row_ptr, int64_t nrows, int s,
                                     int64_t *blk) {
  __shared__ int64_t ws[33];
  int64_t base = (int64_t)blockIdx.x * kSelPerBlock + (int64_t)threadIdx.x * kSelItems;
  int64_t cnt = 0;
#pragma unroll
  for (int k = 0; k < kSelItems; ++k) {
    int64_t u = base + k;
    if (u < nrows) cnt += (row_ptr[u + 1] - row_ptr[u]) >= s;
  }
  int64_t tot;
  block_excl_scan<int64_t>(cnt, ws, &tot);
  if (threadIdx.x == 0) blk[blockIdx.x] = tot;
}

__global__ void sel_csr_write_kernel(const int64_t *__restrict__ row_ptr, int64_t nrows, int s,
                                     int64_t row_lo, const int64_t *__restrict__ blk,
                                     int64_t *rstart, int32_t *rlen, uint32_t *rowid) {
  __shared__ int64_t ws[33];
  int64_t base = (int64_t)blockIdx.x * kSelPerBlock + (int64_t)threadIdx.x * kSelItems;
  int64_t b[kSelItems], d[kSelItems];
  int64_t cnt = 0;
#pragma unroll
  for (int k = 0; k < kSelItems; ++k) {
    int64_t u = base + k;
    d[k] = -1;
    if (u < nrows) {
      b[k] = row_ptr[u];
      d[k] = row_ptr[u + 1] - b[k];
      cnt += d[k] >= s;
    }
  }
  int64_t tot;
  int64_t o = blk[blockIdx.x] + block_excl_scan<int64_t>(cnt, ws, &tot);
#pragma unroll
  for (int k = 0; k < kSelItems; ++k) {
    if (d[k] >= s) {
      rstart[o] = b[k];
      rlen[o] = (int32_t)d[k];
      rowid[o] = (uint32_t)(row_lo + base + k);
      ++o;
    }
  }
}

// ---- pass II selection: groups of G_I with |L| >= s --------------------------
// Thread per 32-bit word of head bits.  A group starting at bit p ends at the
// next head bit (trial segments start with a head, so groups never cross
// trials) or at npairs.
__device__ __forceinline__ int64_t next_head(const uint32_t *__restrict__ head, int64_t nwords,
                                             int64_t npairs, int64_t w, uint32_t rest) {
  // rest: bits of word w above the current head
  if (rest) return (w << 5) + __ffs(rest) - 1;
  for (int64_t x = w + 1; x < nwords; ++x) {
    uint32_t v = head[x];
    if (v) return (x << 5) + __ffs(v) - 1;
  }
  return npairs;
}

__global__ void sel_grp_count_kernel(const uint32_t *__restrict__ head, int64_t npairs, int s,
                                     int64_t *blk) {
  __shared__ int64_t ws[33];
  const int64_t nwords = (npairs + 31) >> 5;
  int64_t base = (int64_t)blockIdx.x * kSelPerBlock + (int64_t)threadIdx.x * kSelItems;
  int64_t cnt = 0;
  for (int k = 0; k < kSelItems; ++k) {
    int64_t w = base + k;
    if (w >= nwords) break;
    uint32_t bits = head[w];
    while (bits) {
      int i = __ffs(bits) - 1;
      bits &= bits - 1;
      int64_t p = (w << 5) + i;
      int64_t q = next_head(head, nwords, npairs, w, bits);
      cnt += (q - p) >= s;
    }
  }
  int64_t tot;
  block_excl_scan<int64_t>(cnt, ws, &tot);
  if (threadIdx.x == 0) blk[blockIdx.x] = tot;
}

__global__ void sel_grp_write_kernel(const uint32_t *__restrict__ head, int64_t npairs, int s,
                                     const int64_t *__restrict__ blk, int64_t *rstart,
                                     int32_t *rlen) {
  __shared__ int64_t ws[33];
  const int64_t nwords = (npairs + 31) >> 5;
  int64_t base = (int64_t)blockIdx.x * kSelPerBlock + (int64_t)threadIdx.x * kSelItems;
  int64_t cnt = 0;
  for (int k = 0; k < kSelItems; ++k) {
    int64_t w = base + k;
    if (w >= nwords) break;
    uint32_t bits = head[w];
    while (bits) {
      int i = __ffs(bits) - 1;
      bits &= bits - 1;
      int64_t p = (w << 5) + i;
      int64_t q = next_head(head, nwords, npairs, w, bits);
      cnt += (q - p) >= s;
    }
  }
  int64_t tot;
  int64_t o = blk[blockIdx.x] + block_excl_scan<int64_t>(cnt, ws, &tot);
  for (int k = 0; k < kSelItems; ++k) {
    int64_t w = base + k;
    if (w >= nwords) break;
    uint32_t bits = head[w];
    while (bits) {
      int i = __ffs(bits) - 1;
      bits &= bits - 1;
      int64_t p = (w << 5) + i;
      int64_t q = next_head(head, nwords, npairs, w, bits);
      if (q - p >= s) {
        rstart[o] = p;
        rlen[o] = (int32_t)(q - p);
        ++o;
      }
    }
  }
}

// ---- multi-rank helpers -------------------------------------------------------
__device__ __forceinline__ int upper_trial(const int64_t *seg, int c, int64_t x) {
  int lo = 0, hi = c;          // last j with seg[j] <= x
  while (hi - lo > 1) {
    const int mid = (lo + hi) >> 1;
    if (seg[mid] <= x) lo = mid;
    else hi = mid;
  }
  return lo;
}

__global__ void rows_per_trial_kernel(const int64_t *__restrict__ rstart, int64_t nrows,
                                      const int64_t *__restrict__ seg, int c,
                                      unsigned long long *counts) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nrows;
       i += (int64_t)gridDim.x * blockDim.x)
    atomicAdd(&counts[upper_trial(seg, c, rstart[i])], 1ull);
}

__global__ void assign_rowid_kernel(uint32_t *rowid, int64_t nrows, const int64_t *__restrict__ first,
                                    const int64_t *__restrict__ off, int c) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nrows;
       i += (int64_t)gridDim.x * blockDim.x)
    rowid[i] = (uint32_t)(i + off[upper_trial(first, c, i)]);
}

}  // namespace

int64_t sel_scratch_elems(int64_t items) { return (items + kSelPerBlock - 1) / kSelPerBlock + 1; }

cudaError_t select_csr_count(const int64_t *row_ptr, int64_t nrows, int s, int64_t *blk,
                             int64_t *d_total, cudaStream_t st) {
  int64_t nb = (nrows + kSelPerBlock - 1) / kSelPerBlock;
  if (nb > 0) {
    sel_csr_count_kernel<<<(unsigned)nb, kSelThreads, 0, st>>>(row_ptr, nrows, s, blk);
    ++g_launches;
  }
  scan_inplace_kernel<<<1, 1024, 0, st>>>(blk, nb, d_total);
  ++g_launches;
  return cudaGetLastError();
}

cudaError_t select_csr_write(const int64_t *row_ptr, int64_t nrows, int s, int64_t row_lo,
                             const int64_t *blk, int64_t *rstart, int32_t *rlen, uint32_t *rowid,
                             cudaStream_t st) {
  int64_t nb = (nrows + kSelPerBlock - 1) / kSelPerBlock;
  if (nb > 0)
    {
    sel_csr_write_kernel<<<(unsigned)nb, kSelThreads, 0, st>>>(row_ptr, nrows, s, row_lo, blk,
                                                               rstart, rlen, rowid);
    ++g_launches;
  }
  return cudaGetLastError();
}

cudaError_t select_groups_count(const uint32_t *head, int64_t npairs, int s, int64_t *blk,
                                int64_t *d_total, cudaStream_t st) {
  int64_t nwords = (npairs + 31) >> 5;
  int64_t nb = (nwords + kSelPerBlock - 1) / kSelPerBlock;
  if (nb > 0) {
    sel_grp_count_kernel<<<(unsigned)nb, kSelThreads, 0, st>>>(head, npairs, s, blk);
    ++g_launches;
  }
  scan_inplace_kernel<<<1, 1024, 0, st>>>(blk, nb, d_total);
  ++g_launches;
  return cudaGetLastError();
}

cudaError_t select_groups_write(const uint32_t *head, int64_t npairs, int s, const int64_t *blk,
                                int64_t *rstart, int32_t *rlen, cudaStream_t st) {
  int64_t nwords = (npairs + 31) >> 5;
  int64_t nb = (nwords + kSelPerBlock - 1) / kSelPerBlock;
  if (nb > 0)
    {
    sel_grp_write_kernel<<<(unsigned)nb, kSelThreads, 0, st>>>(head, npairs, s, blk, rstart, rlen);
    ++g_launches;
  }
  return cudaGetLastError();
}


cudaError_t rows_per_trial(const int64_t *rstart, int64_t nrows, const int64_t *seg, int32_t c,
                           unsigned long long *counts, cudaStream_t st) {
  if (nrows == 0) return cudaSuccess;
  const int grid = (int)std::min<int64_t>((nrows + 255) / 256, 148 * 8);
  rows_per_trial_kernel<<<grid, 256, 0, st>>>(rstart, nrows, seg, c, counts);
  ++g_launches;
  return cudaGetLastError();
}

cudaError_t assign_rowid(uint32_t *rowid, int64_t nrows, const int64_t *first, const int64_t *off,
                         int32_t c, cudaStream_t st) {
  if (nrows == 0) return cudaSuccess;
  const int grid = (int)std::min<int64_t>((nrows + 255) / 256, 148 * 8);
  assign_rowid_kernel<<<grid, 256, 0, st>>>(rowid, nrows, first, off, c);
  ++g_launches;
  return cudaGetLastError();
}

}  // namespace sg
