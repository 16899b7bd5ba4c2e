// kernels_pass.cu — row selection and the per-row top-s min-hash (one
// shingling pass; Alg. 1) for sm_100a.
//
// Design: the paper hashes every adjacency entry into a
// materialised copy and segment-sorts it once per trial (Alg. 1 l.8-17).  On
// B200 the pass is integer-ALU bound, so nothing is materialised: one warp
// owns a row, stages its adjacency list once in shared memory and reuses it
// for all c trials; each lane owns a trial (lane = trial, neighbours
// broadcast from smem as 128-bit words) and keeps its s minima in registers
// (the paper's insertion-sorted s-array).  When c is not a
// multiple of 32 the tail trials are split across lanes by neighbour subsets
// and merged with warp shuffles.  Output: key = fmix(id) trial-major.
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

// ---- min-hash top-s ----------------------------------------------------------
constexpr int kMhThreads = 256;
constexpr int kMhWarps = kMhThreads / 32;
constexpr int kNbCap = 1024;        // staged neighbours per warp (4 KB)
constexpr int kMaxPasses = 48;

struct TrialPass {
  int16_t t0;      // first trial of the pass
  int8_t logT;     // trials in the pass = 2^logT (lane & (T-1))
  int8_t logp;     // neighbour parts = 2^logp (lane >> logT); T * p = 32 or T < 32, p = 1
};

struct MhParams {
  MinhashArgs a;
  int32_t npass;
  int32_t rows_per_grab;
  TrialPass pass[kMaxPasses];
};

// Keep the S smallest values of m[] U {h}, ascending (the paper's s-array
// with insertion); branch-free compare-exchange chain.
template <int S>
__device__ __forceinline__ void insert_min(uint32_t (&m)[S], uint32_t h) {
#pragma unroll
  for (int i = 0; i < S; ++i) {
    uint32_t lo = min(m[i], h);
    h = max(m[i], h);
    m[i] = lo;
  }
}

template <int S>
__device__ __forceinline__ uint64_t shingle_id(const uint32_t (&m)[S], uint64_t seed, int j) {
  if (S == 1) return (uint64_t)m[0];
  if (S == 2) return ((uint64_t)m[0] << 31) | (uint64_t)m[S - 1];
  uint64_t z = fmix(seed ^ fmix((uint64_t)j + 1));
#pragma unroll
  for (int i = 0; i < S; ++i) z = fmix(z + (uint64_t)m[i]);
  return z;
}

// Scan entries nb[e] for e = part, part + p, ... < len.
template <int S>
__device__ __forceinline__ void scan_strided(const uint32_t *nb, int len, int part, int p,
                                             uint32_t a, uint32_t b, uint32_t (&m)[S]) {
  for (int e = part; e < len; e += p) {
    uint32_t h = m31_hash(a, b, nb[e]);
    if (h < m[S - 1]) insert_min<S>(m, h);
  }
}

// p == 1: every lane scans all entries; 128-bit broadcast loads from smem.
template <int S>
__device__ __forceinline__ void scan_all(const uint32_t *nb, int len, uint32_t a, uint32_t b,
                                         uint32_t (&m)[S]) {
  const uint4 *nb4 = reinterpret_cast<const uint4 *>(nb);
  int len4 = len >> 2;
#pragma unroll 2
  for (int q = 0; q < len4; ++q) {
    uint4 v = nb4[q];
    uint32_t h0 = m31_hash(a, b, v.x);
    uint32_t h1 = m31_hash(a, b, v.y);
    uint32_t h2 = m31_hash(a, b, v.z);
    uint32_t h3 = m31_hash(a, b, v.w);
    uint32_t hm = min(min(h0, h1), min(h2, h3));
    if (hm < m[S - 1]) {
      insert_min<S>(m, h0);
      insert_min<S>(m, h1);
      insert_min<S>(m, h2);
      insert_min<S>(m, h3);
    }
  }
  for (int e = len4 << 2; e < len; ++e) {
    uint32_t h = m31_hash(a, b, nb[e]);
    if (h < m[S - 1]) insert_min<S>(m, h);
  }
}

template <int S>
__global__ void __launch_bounds__(kMhThreads) minhash_warp_kernel(const __grid_constant__ MhParams P) {
  extern __shared__ __align__(16) uint32_t smem[];
  const MinhashArgs &a = P.a;
  const int c = a.c;
  const int cpad = (c + 3) & ~3;
  uint32_t *sA = smem;
  uint32_t *sB = smem + cpad;
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  uint32_t *nb = smem + 2 * cpad + wid * kNbCap;
  for (int i = threadIdx.x; i < c; i += blockDim.x) {
    sA[i] = a.A[i];
    sB[i] = a.B[i];
  }
  __syncthreads();
  const int64_t nrows = a.nrows;
  for (;;) {
    unsigned long long r0 = 0;
    if (lane == 0) r0 = atomicAdd(a.counter, (unsigned long long)P.rows_per_grab);
    r0 = __shfl_sync(0xffffffffu, r0, 0);
    if ((int64_t)r0 >= nrows) break;
    int64_t r1 = min((int64_t)r0 + P.rows_per_grab, nrows);
    for (int64_t r = (int64_t)r0; r < r1; ++r) {
      const int64_t st = a.rstart[r];
      const int len = a.rlen[r];
      const uint32_t *__restrict__ src = a.entries + st;
      const bool staged = len <= kNbCap;
      __syncwarp();
      if (staged) {
        for (int i = lane; i < len; i += 32) nb[i] = src[i];
        __syncwarp();
      }
      for (int pi = 0; pi < P.npass; ++pi) {
        const TrialPass tp = P.pass[pi];
        const int T = 1 << tp.logT;
        const int p = 1 << tp.logp;
        const int tl = lane & (T - 1);
        const int part = lane >> tp.logT;
        const int j = tp.t0 + tl;
        const bool live = (lane < T * p);
        const uint32_t A = sA[min(j, c - 1)], B = sB[min(j, c - 1)];
        uint32_t m[S];
#pragma unroll
        for (int i = 0; i < S; ++i) m[i] = 0xFFFFFFFFu;
        if (staged) {
          if (live) {
            if (p == 1) scan_all<S>(nb, len, A, B, m);
            else scan_strided<S>(nb, len, part, p, A, B, m);
          }
        } else {
          for (int c0 = 0; c0 < len; c0 += kNbCap) {
            const int cl = min(kNbCap, len - c0);
            __syncwarp();
            for (int i = lane; i < cl; i += 32) nb[i] = src[c0 + i];
            __syncwarp();
            if (live) {
              if (p == 1) scan_all<S>(nb, cl, A, B, m);
              else scan_strided<S>(nb, cl, part, p, A, B, m);
            }
          }
        }
        // merge the p partial top-s lists of a trial (lanes tl, tl+T, ...)
        for (int o = T; o < 32; o <<= 1) {
          uint32_t x[S];
#pragma unroll
          for (int i = 0; i < S; ++i) x[i] = __shfl_xor_sync(0xffffffffu, m[i], o);
#pragma unroll
          for (int i = 0; i < S; ++i) insert_min<S>(m, x[i]);
        }
        if (live && part == 0) {
          a.keys[(int64_t)j * nrows + r] = fmix(shingle_id<S>(m, a.seed, j));
        }
      }
    }
  }
}

template <int S>
cudaError_t launch_minhash(const MhParams &P, int num_sms, cudaStream_t st) {
  const int cpad = (P.a.c + 3) & ~3;
  size_t smem = (size_t)(2 * cpad + kMhWarps * kNbCap) * sizeof(uint32_t);
  auto kern = minhash_warp_kernel<S>;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  int per_sm = 0;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, kMhThreads, smem);
  if (e != cudaSuccess) return e;
  if (per_sm < 1) per_sm = 1;
  int64_t want = (P.a.nrows + kMhWarps - 1) / kMhWarps;
  int grid = (int)std::min<int64_t>((int64_t)num_sms * per_sm, std::max<int64_t>(want, 1));
  kern<<<grid, kMhThreads, smem, st>>>(P);
  ++g_launches;
  return cudaGetLastError();
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

cudaError_t minhash(const MinhashArgs &a, int num_sms, cudaStream_t st) {
  if (a.nrows == 0) return cudaSuccess;
  MhParams P;
  P.a = a;
  // trial passes: full groups of 32 lanes (one trial per lane), then the
  // binary digits of c mod 32 (2^b trials x 32/2^b neighbour parts)
  int np = 0, t = 0;
  while (a.c - t >= 32) {
    P.pass[np++] = TrialPass{(int16_t)t, 5, 0};
    t += 32;
  }
  for (int b = 4; b >= 0; --b) {
    if ((a.c - t) & (1 << b)) {
      P.pass[np++] = TrialPass{(int16_t)t, (int8_t)b, (int8_t)(5 - b)};
      t += 1 << b;
    }
  }
  P.npass = np;
  int64_t warps = (int64_t)num_sms * 48;
  P.rows_per_grab = (int32_t)std::max<int64_t>(1, std::min<int64_t>(64, a.nrows / (warps * 16)));
  switch (a.s) {
    case 1: return launch_minhash<1>(P, num_sms, st);
    case 2: return launch_minhash<2>(P, num_sms, st);
    case 3: return launch_minhash<3>(P, num_sms, st);
    case 4: return launch_minhash<4>(P, num_sms, st);
    case 5: return launch_minhash<5>(P, num_sms, st);
    case 6: return launch_minhash<6>(P, num_sms, st);
    case 7: return launch_minhash<7>(P, num_sms, st);
    case 8: return launch_minhash<8>(P, num_sms, st);
    default: return cudaErrorInvalidValue;
  }
}

}  // namespace sg
