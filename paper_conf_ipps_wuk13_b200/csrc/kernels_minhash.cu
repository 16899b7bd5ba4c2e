// kernels_minhash.cu — the per-row top-s min-hash of one shingling pass
// (Alg. 1) for sm_100a.
//
// The paper hashes every adjacency entry into a materialised copy and
// segment-sorts it once per trial (Alg. 1 l.8-17).  On B200 the pass is
// integer-ALU bound, so nothing is materialised:
//  * a warp owns a tile of 8 consecutive rows and stages their adjacency
//    lists once in shared memory (concatenated, 16 B aligned);
//  * lane = trial: 32 trials run side by side on the same neighbour,
//    broadcast from smem as 128-bit words; the s minima live in registers
//    (the paper's insertion-sorted s-array);
//  * when c is not a multiple of 32, the tail trials are split over lanes by
//    neighbour subsets and merged with warp shuffles;
//  * h = (A v + B) mod (2^31 - 1): one IMAD.WIDE + Mersenne fold + one
//    conditional subtract (sg_internal.cuh);
//  * each lane ends a tile with the 8 keys of its trial for 8 consecutive
//    rows: one 64 B (two full sectors) store into the trial-major key array.
#include <algorithm>

#include "kernels.h"
#include "scan.cuh"
#include "sg_internal.cuh"

namespace sg {

namespace {

constexpr int kMhThreads = 256;
constexpr int kMhWarps = kMhThreads / 32;
// Rows longer than this (hub vertices) are left to the block-per-vertex
// hub_kernel: one CTA per row, the row split over its 8 warps.
constexpr int kHubLen = 2048;

// staged entries per warp: 4 KB for 8-row tiles of long rows, 2 KB for
// 16-row tiles of short rows (the 16-row key buffer takes the difference)
template <int TR>
__host__ __device__ constexpr int nb_cap() { return TR == 8 ? 1024 : 512; }
constexpr int kMaxPasses = 48;

struct TrialPass {
  int16_t t0;      // first trial of the pass (relative to the launch's t0)
  int8_t logT;     // trials in the pass = 2^logT  (trial = lane & (T-1))
  int8_t logp;     // neighbour parts    = 2^logp  (part  = lane >> logT)
};

struct MhParams {
  MinhashArgs a;
  int32_t npass;
  int32_t tiles_per_grab;
  TrialPass pass[kMaxPasses];
};

// Keep the S smallest of m[] U {h} ascending: compare-exchange chain.
template <int S>
__device__ __forceinline__ void insert_min(uint32_t (&m)[S], uint32_t h) {
#pragma unroll
  for (int i = 0; i < S; ++i) {
    uint32_t lo = min(m[i], h);
    h = max(m[i], h);
    m[i] = lo;
  }
}

// Within-trial shingle id (AMB-4).
template <int S>
__device__ __forceinline__ uint64_t shingle_id(const uint32_t (&m)[S], uint64_t seed, int j) {
  if (S == 1) return (uint64_t)m[0];
  if (S == 2) return ((uint64_t)m[0] << 31) | (uint64_t)m[S - 1];
  uint64_t z = fmix(seed ^ fmix((uint64_t)j + 1));
#pragma unroll
  for (int i = 0; i < S; ++i) z = fmix(z + (uint64_t)m[i]);
  return z;
}

template <int S>
__device__ __forceinline__ void scan_strided(const uint32_t *nb, int len, int part, int p,
                                             uint32_t a, uint32_t b, uint32_t (&m)[S]) {
  for (int e = part; e < len; e += p) {
    uint32_t h = m31_hash(a, b, nb[e]);
    if (h < m[S - 1]) insert_min<S>(m, h);
  }
}

// p == 1: every lane scans every entry, 4 per 128-bit broadcast load.
template <int S>
__device__ __forceinline__ void scan_all(const uint32_t *nb, int len, uint32_t a, uint32_t b,
                                         uint32_t (&m)[S]) {
  const uint4 *nb4 = reinterpret_cast<const uint4 *>(nb);
  const int len4 = len >> 2;
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

// Short rows (pass-II rows average ~5 entries): whole quads branch-free, then
// the 0-3 remaining entries as one pair and one single (row length is
// warp-uniform: every lane scans the same row for its own trial), so no
// padding slot is ever hashed.
template <int S>
__device__ __forceinline__ void scan_short(const uint32_t *nb, int len, uint32_t a, uint32_t b,
                                           uint32_t (&m)[S]) {
  const uint4 *nb4 = reinterpret_cast<const uint4 *>(nb);
  int q = 0;
  for (; q + 4 <= len; q += 4) {
    const uint4 v = nb4[q >> 2];
    insert_min<S>(m, m31_hash(a, b, v.x));
    insert_min<S>(m, m31_hash(a, b, v.y));
    insert_min<S>(m, m31_hash(a, b, v.z));
    insert_min<S>(m, m31_hash(a, b, v.w));
  }
  if (len - q >= 2) {
    const uint2 v = reinterpret_cast<const uint2 *>(nb)[q >> 1];
    insert_min<S>(m, m31_hash(a, b, v.x));
    insert_min<S>(m, m31_hash(a, b, v.y));
    q += 2;
  }
  if (q < len) insert_min<S>(m, m31_hash(a, b, nb[q]));
}

constexpr uint32_t kPad = 0xFFFFFFFFu;   // staged padding (vertex ids are < P < 2^31)

// h of a staged word; padding words hash to all-ones (never among the minima)
__device__ __forceinline__ uint32_t hash_or_pad(uint32_t A, uint32_t B, uint32_t v) {
  return m31_hash(A, B, v) | (uint32_t)((int32_t)v >> 31);
}

// Two rows of na / nb (<= 4, warp-uniform) padded pairs, scanned side by
// side: 64-bit broadcast loads, so a 2-entry row hashes 2 slots, not 4.
// (Hashing the odd entry alone instead of testing for the padding word was
// measured slower: 11.05e9 vs 10.87e9 instructions per 64-trial chunk.)
template <int S>
__device__ __forceinline__ void pairs2(const uint32_t *pa, const uint32_t *pb, int na, int nb,
                                       uint32_t A, uint32_t B, uint32_t (&ma)[S], uint32_t (&mb)[S]) {
  const uint2 *a2 = reinterpret_cast<const uint2 *>(pa);
  const uint2 *b2 = reinterpret_cast<const uint2 *>(pb);
#pragma unroll
  for (int q = 0; q < 4; ++q) {
    if (q < na) {
      const uint2 v = a2[q];
      insert_min<S>(ma, hash_or_pad(A, B, v.x));
      insert_min<S>(ma, hash_or_pad(A, B, v.y));
    }
    if (q < nb) {
      const uint2 v = b2[q];
      insert_min<S>(mb, hash_or_pad(A, B, v.x));
      insert_min<S>(mb, hash_or_pad(A, B, v.y));
    }
  }
}

template <int S>
__device__ __forceinline__ void scan_any(const uint32_t *nb, int len, int part, int p, uint32_t a,
                                         uint32_t b, uint32_t (&m)[S]) {
  if (p == 1) scan_all<S>(nb, len, a, b, m);
  else scan_strided<S>(nb, len, part, p, a, b, m);
}

// Per-warp key buffer slot of (row rr, trial lane tt): rows in 32-slot lines,
// lanes XOR-swizzled by the row pair so that the coalesced store's reads of
// one trial's rows fall in distinct banks.
__device__ __forceinline__ int out_slot(int rr, int tt) { return rr * 32 + (tt ^ (rr >> 1)); }

template <int S, int TR>
__global__ void __launch_bounds__(kMhThreads, 4) minhash_tile_kernel(const __grid_constant__ MhParams P) {
  extern __shared__ __align__(16) unsigned char smraw[];
  __shared__ int64_t sSt[kMhWarps][TR];
  __shared__ __align__(16) int sLen[kMhWarps][TR + 4];   // [TR]: read-ahead pad
  __shared__ __align__(16) int sOff[kMhWarps][TR + 8];   // 16 B aligned rows
  const MinhashArgs &a = P.a;
  const int nt = a.nt;
  const int ntp = (nt + 7) & ~7;
  uint32_t *sA = reinterpret_cast<uint32_t *>(smraw);
  uint32_t *sB = sA + ntp;
  uint64_t *sOutAll = reinterpret_cast<uint64_t *>(sB + ntp);
  uint32_t *sNbAll = reinterpret_cast<uint32_t *>(sOutAll + kMhWarps * TR * 32);
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  uint64_t *sOut = sOutAll + w * TR * 32;
  uint32_t *nb = sNbAll + w * nb_cap<TR>();
  for (int i = threadIdx.x; i < nt; i += blockDim.x) {
    sA[i] = a.A[a.t0 + i];
    sB[i] = a.B[a.t0 + i];
  }
  __syncthreads();
  const int64_t nrows = a.nrows;
  const int64_t ntiles = (nrows + TR - 1) / TR;
  for (;;) {
    unsigned long long g0 = 0;
    if (lane == 0) g0 = atomicAdd(a.counter, (unsigned long long)P.tiles_per_grab);
    g0 = __shfl_sync(0xffffffffu, g0, 0);
    if ((int64_t)g0 >= ntiles) break;
    const int64_t g1 = min((int64_t)g0 + P.tiles_per_grab, ntiles);
    for (int64_t tile = (int64_t)g0; tile < g1; ++tile) {
      const int64_t r0 = tile * TR;
      const int nr = (int)min((int64_t)TR, nrows - r0);
      __syncwarp();
      int len = 0;
      int64_t st = 0;
      if (lane < nr) {
        st = a.rstart[r0 + lane];
        len = a.rlen[r0 + lane];
      }
      const int plen = (len + 3) & ~3;
      const int incl = warp_incl_scan(plen);
      if (lane < TR) {
        sSt[w][lane] = st;
        sLen[w][lane] = len;
        sOff[w][lane + 1] = incl;
      }
      if (lane == 0) sOff[w][0] = 0;
      __syncwarp();
      const int total = sOff[w][TR];
      if (total > nb_cap<TR>()) {
        // long rows: one row at a time, staged once (or chunk by chunk when it
        // exceeds the stage), all trial passes on it, scalar key stores
        for (int rr = 0; rr < nr; ++rr) {
          const int rl = sLen[w][rr];
          if (rl > kHubLen) continue;                 // block-per-vertex kernel (hub_kernel)
          const uint32_t *src = a.entries + sSt[w][rr];
          const bool fits = rl <= nb_cap<TR>();
          if (fits) {
            __syncwarp();
            for (int i = lane; i < rl; i += 32) nb[i] = src[i];
            __syncwarp();
          }
          for (int pi = 0; pi < P.npass; ++pi) {
            const TrialPass tp = P.pass[pi];
            const int T = 1 << tp.logT;
            const int p = 1 << tp.logp;
            const int tl = lane & (T - 1);
            const int part = lane >> tp.logT;
            const int j = tp.t0 + tl;
            const uint32_t A = sA[j], B = sB[j];
            uint32_t m[S];
#pragma unroll
            for (int i = 0; i < S; ++i) m[i] = 0xFFFFFFFFu;
            if (fits) {
              scan_any<S>(nb, rl, part, p, A, B, m);
            } else {
              for (int c0 = 0; c0 < rl; c0 += nb_cap<TR>()) {
                const int cl = min(nb_cap<TR>(), rl - c0);
                __syncwarp();
                for (int i = lane; i < cl; i += 32) nb[i] = src[c0 + i];
                __syncwarp();
                scan_any<S>(nb, cl, part, p, A, B, m);
              }
            }
            for (int o = T; o < 32; o <<= 1) {
              uint32_t x[S];
#pragma unroll
              for (int i = 0; i < S; ++i) x[i] = __shfl_xor_sync(0xffffffffu, m[i], o);
#pragma unroll
              for (int i = 0; i < S; ++i) insert_min<S>(m, x[i]);
            }
            if (part == 0) {
              const uint64_t key = fmix(shingle_id<S>(m, a.seed, a.t0 + j));
              a.keys[(int64_t)j * a.key_stride + r0 + rr] = key;
              if (a.kbin) a.kbin[(int64_t)j * a.key_stride + r0 + rr] = (uint8_t)(key >> 56);
            }
          }
        }
        continue;
      }
      // short rows: the whole tile staged once, trial passes outer, rows inner
      for (int i = lane; i < total; i += 32) {
        int rr = 0;
#pragma unroll
        for (int x = 1; x < TR; ++x) rr += (i >= sOff[w][x]);
        const int k = i - sOff[w][rr];
        nb[i] = k < sLen[w][rr] ? a.entries[sSt[w][rr] + k] : kPad;   // pad: all-ones
      }
      __syncwarp();
      for (int pi = 0; pi < P.npass; ++pi) {
        const TrialPass tp = P.pass[pi];
        const int T = 1 << tp.logT;
        const int p = 1 << tp.logp;
        const int tl = lane & (T - 1);
        const int part = lane >> tp.logT;
        const int j = tp.t0 + tl;               // trial index within the launch
        const uint32_t A = sA[j], B = sB[j];
        if (p == 1) {
          // full 32-trial pass: rows of <= 8 entries go in pairs, straight-line
          // over their padded quads (two independent chains per lane)
          int rr = 0;
          while (rr < nr) {
            const int la = sLen[w][rr];
            const int lb = rr + 1 < nr ? sLen[w][rr + 1] : 1 << 30;
            if (la <= 8 && lb <= 8) {
              const uint32_t *pa = nb + sOff[w][rr], *pb = nb + sOff[w][rr + 1];
              uint32_t ma[S], mb[S];
#pragma unroll
              for (int i = 0; i < S; ++i) ma[i] = mb[i] = 0xFFFFFFFFu;
              pairs2<S>(pa, pb, (la + 1) >> 1, (lb + 1) >> 1, A, B, ma, mb);
              sOut[out_slot(rr, lane)] = fmix(shingle_id<S>(ma, a.seed, a.t0 + j));
              sOut[out_slot(rr + 1, lane)] = fmix(shingle_id<S>(mb, a.seed, a.t0 + j));
              rr += 2;
            } else {
              uint32_t m[S];
#pragma unroll
              for (int i = 0; i < S; ++i) m[i] = 0xFFFFFFFFu;
              if (la <= 24) scan_short<S>(nb + sOff[w][rr], la, A, B, m);
              else scan_all<S>(nb + sOff[w][rr], la, A, B, m);
              sOut[out_slot(rr, lane)] = fmix(shingle_id<S>(m, a.seed, a.t0 + j));
              rr += 1;
            }
          }
        } else if (TR == 16) {
          // tail pass over short rows: the p lane groups take different rows
          // (row rr = rb + part), each lane scanning a whole row for its trial
          for (int rb = 0; rb < nr; rb += p) {
            const int rr = rb + part;
            if (rr < nr) {
              const int rl = sLen[w][rr];
              uint32_t m[S];
#pragma unroll
              for (int i = 0; i < S; ++i) m[i] = 0xFFFFFFFFu;
              if (rl <= 24) scan_short<S>(nb + sOff[w][rr], rl, A, B, m);
              else scan_all<S>(nb + sOff[w][rr], rl, A, B, m);
              sOut[out_slot(rr, tl)] = fmix(shingle_id<S>(m, a.seed, a.t0 + j));
            }
          }
        } else {
        int rl_n = sLen[w][0], ro_n = sOff[w][0];   // row rr's metadata, loaded a row ahead
        for (int rr = 0; rr < nr; ++rr) {
          const int rl = rl_n;
          const uint32_t *rnb = nb + ro_n;
          rl_n = sLen[w][rr + 1];
          ro_n = sOff[w][rr + 1];
          uint32_t m[S];
#pragma unroll
          for (int i = 0; i < S; ++i) m[i] = 0xFFFFFFFFu;
          if (p == 1 && rl <= 24) scan_short<S>(rnb, rl, A, B, m);
          else scan_any<S>(rnb, rl, part, p, A, B, m);
          // merge the p partial lists of a trial (lanes tl, tl + T, ...)
          for (int o = T; o < 32; o <<= 1) {
            uint32_t x[S];
#pragma unroll
            for (int i = 0; i < S; ++i) x[i] = __shfl_xor_sync(0xffffffffu, m[i], o);
#pragma unroll
            for (int i = 0; i < S; ++i) insert_min<S>(m, x[i]);
          }
          if (part == 0) sOut[out_slot(rr, tl)] = fmix(shingle_id<S>(m, a.seed, a.t0 + j));
        }
        }
        __syncwarp();
        // coalesced stores: a trial's TR keys are TR * 8 contiguous bytes of
        // its segment; consecutive lanes take consecutive 16 B pieces
        if (nr == TR) {
          constexpr int CPT = TR / 2;            // 16 B pieces per trial
#pragma unroll
          for (int q = 0; q < CPT; ++q) {
            const int c = q * 32 + lane;
            const int tt = c / CPT, pp = c % CPT;
            if (tt < T) {
              const uint64_t k0 = sOut[out_slot(2 * pp, tt)], k1 = sOut[out_slot(2 * pp + 1, tt)];
              *reinterpret_cast<ulonglong2 *>(a.keys + (int64_t)(tp.t0 + tt) * a.key_stride + r0 +
                                              2 * pp) = make_ulonglong2(k0, k1);
            }
          }
          if (a.kbin && lane < T) {
            // the tile's TR top key bytes of trial `lane`: one TR-byte store
            const uint32_t *hi = reinterpret_cast<const uint32_t *>(sOut);
            uint32_t w[TR / 4];
#pragma unroll
            for (int q = 0; q < TR / 4; ++q) {
              w[q] = 0;
#pragma unroll
              for (int x = 0; x < 4; ++x)
                w[q] |= (hi[2 * out_slot(4 * q + x, lane) + 1] >> 24) << (8 * x);
            }
            uint8_t *bd = a.kbin + (int64_t)(tp.t0 + lane) * a.key_stride + r0;
            if (TR == 16) *reinterpret_cast<uint4 *>(bd) = make_uint4(w[0], w[1], w[2], w[3]);
            else *reinterpret_cast<uint2 *>(bd) = make_uint2(w[0], w[1]);
          }
        } else if (part == 0) {
          uint64_t *dst = a.keys + (int64_t)j * a.key_stride + r0;
          for (int rr = 0; rr < nr; ++rr) dst[rr] = sOut[out_slot(rr, tl)];
          if (a.kbin)
            for (int rr = 0; rr < nr; ++rr)
              a.kbin[(int64_t)j * a.key_stride + r0 + rr] = (uint8_t)(sOut[out_slot(rr, tl)] >> 56);
        }
        __syncwarp();
      }
    }
  }
}

// Block-per-vertex min-hash of hub rows (len > kHubLen): the CTA scans its
// share of the rows' lengths; each hub found is processed by the whole CTA.
// The row is staged in shared memory (kHubStage entries at a time,
// coalesced) and every trial pass reads it from there: warp w takes the w-th
// eighth of the staged quads, lane = trial (full passes) or (trial,
// neighbour part) (tail passes), 128-bit broadcast loads, four hashes per
// load; the eight partial top-s lists of a trial are merged through shared
// memory.  Rows longer than the stage are re-staged per pass.
constexpr int kHubStage = 16384;                 // entries (64 KB)

template <int S>
__global__ void __launch_bounds__(kMhThreads) hub_kernel(const __grid_constant__ MhParams P) {
  extern __shared__ __align__(16) unsigned char smraw[];
  uint32_t *stg = reinterpret_cast<uint32_t *>(smraw);
  __shared__ uint32_t sPart[kMhWarps][32][S];
  __shared__ int sHub[kMhThreads];
  __shared__ int sNHub;
  const MinhashArgs &a = P.a;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  __shared__ int64_t sB0;
  for (;;) {
    // row blocks grabbed dynamically (hubs are few and unevenly spread)
    if (threadIdx.x == 0) {
      sNHub = 0;
      sB0 = (int64_t)atomicAdd(a.hub_counter, 1ull) * kMhThreads;
    }
    __syncthreads();
    const int64_t b0 = sB0;
    if (b0 >= a.nrows) break;
    const int64_t r = b0 + threadIdx.x;
    if (r < a.nrows && a.rlen[r] > kHubLen) sHub[atomicAdd(&sNHub, 1)] = threadIdx.x;
    __syncthreads();
    const int nh = sNHub;
    for (int hI = 0; hI < nh; ++hI) {
      const int64_t row = b0 + sHub[hI];
      const int len = a.rlen[row];
      const uint32_t *src = a.entries + a.rstart[row];
      const bool once = len <= kHubStage;
      if (once) {
        __syncthreads();
        for (int i = threadIdx.x; i < len; i += kMhThreads) stg[i] = src[i];
        __syncthreads();
      }
      for (int pi = 0; pi < P.npass; ++pi) {
        const TrialPass tp = P.pass[pi];
        const int T = 1 << tp.logT;
        const int p = 1 << tp.logp;
        const int tl = lane & (T - 1);
        const int part = lane >> tp.logT;
        const int j = tp.t0 + tl;
        const uint32_t A = a.A[a.t0 + j], B = a.B[a.t0 + j];
        uint32_t m[S];
#pragma unroll
        for (int i = 0; i < S; ++i) m[i] = 0xFFFFFFFFu;
        for (int c0 = 0; c0 < len; c0 += kHubStage) {
          const int cl = min(kHubStage, len - c0);
          if (!once) {
            __syncthreads();
            for (int i = threadIdx.x; i < cl; i += kMhThreads) stg[i] = src[c0 + i];
            __syncthreads();
          }
          const int nq = cl >> 2;
          const int q0 = nq * w / kMhWarps, q1 = nq * (w + 1) / kMhWarps;
          const uint4 *s4 = reinterpret_cast<const uint4 *>(stg);
#pragma unroll 2
          for (int q = q0 + part; q < q1; q += p) {
            const uint4 v = s4[q];
            const uint32_t h0 = m31_hash(A, B, v.x), h1 = m31_hash(A, B, v.y);
            const uint32_t h2 = m31_hash(A, B, v.z), h3 = m31_hash(A, B, v.w);
            if (min(min(h0, h1), min(h2, h3)) < m[S - 1]) {
              insert_min<S>(m, h0);
              insert_min<S>(m, h1);
              insert_min<S>(m, h2);
              insert_min<S>(m, h3);
            }
          }
          if (w == kMhWarps - 1)                        // the 0-3 entries after the last quad
            for (int e = (nq << 2) + part; e < cl; e += p) insert_min<S>(m, m31_hash(A, B, stg[e]));
        }
        for (int o = T; o < 32; o <<= 1) {
          uint32_t x[S];
#pragma unroll
          for (int i = 0; i < S; ++i) x[i] = __shfl_xor_sync(0xffffffffu, m[i], o);
#pragma unroll
          for (int i = 0; i < S; ++i) insert_min<S>(m, x[i]);
        }
#pragma unroll
        for (int i = 0; i < S; ++i) sPart[w][lane][i] = m[i];
        __syncthreads();
        if (w == 0 && part == 0) {
          for (int x = 1; x < kMhWarps; ++x)
#pragma unroll
            for (int i = 0; i < S; ++i) insert_min<S>(m, sPart[x][lane][i]);
          const uint64_t key = fmix(shingle_id<S>(m, a.seed, a.t0 + j));
          a.keys[(int64_t)j * a.key_stride + row] = key;
          if (a.kbin) a.kbin[(int64_t)j * a.key_stride + row] = (uint8_t)(key >> 56);
        }
        __syncthreads();
      }
    }
    __syncthreads();
  }
}

template <int S, int TR>
cudaError_t launch_tile(MhParams &P, int num_sms, cudaStream_t st) {
  const int ntp = (P.a.nt + 7) & ~7;
  const size_t smem = (size_t)2 * ntp * 4 + (size_t)kMhWarps * TR * 32 * 8 +
                      (size_t)kMhWarps * nb_cap<TR>() * 4;
  auto kern = minhash_tile_kernel<S, TR>;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  int per_sm = 0;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, kMhThreads, smem);
  if (e != cudaSuccess) return e;
  per_sm = std::max(per_sm, 1);
  const int64_t ntiles = (P.a.nrows + TR - 1) / TR;
  const int64_t warps = (int64_t)num_sms * 32;
  P.tiles_per_grab = (int32_t)std::max<int64_t>(1, std::min<int64_t>(16, ntiles / (warps * 8)));
  const int64_t want = (ntiles + kMhWarps - 1) / kMhWarps;
  const int grid = (int)std::min<int64_t>((int64_t)num_sms * per_sm, std::max<int64_t>(want, 1));
  kern<<<grid, kMhThreads, smem, st>>>(P);
  ++g_launches;
  if ((e = cudaGetLastError()) != cudaSuccess) return e;
  // hub rows (block per vertex); the tile kernel skipped them
  const size_t hsm = (size_t)kHubStage * 4;
  if ((e = cudaFuncSetAttribute(hub_kernel<S>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                (int)hsm)) != cudaSuccess)
    return e;
  hub_kernel<S><<<num_sms * 3, kMhThreads, hsm, st>>>(P);
  ++g_launches;
  return cudaGetLastError();
}

// ---- pass II, windowed row-per-lane (default for 16-row-tile passes) --------
// The tile kernel gives every (row, trial) of a ~5-entry pass-II row the
// per-row costs of a lane = trial scan (row metadata, staging, loop control:
// ~134 instructions per (row, trial)).  Here a CTA takes a
// window of 256 consecutive rows and sorts them by length class in shared
// memory; warp w takes the w-th 32 rows of that order, one row per lane,
// with the row's <= 8 entries in registers and each trial's (A, B) a
// shared-memory broadcast (lengths agree inside a warp except at the class
// boundaries).  Rows of 9..kHubLen entries are taken one at a time by a
// warp, lane = trial.  The keys of one 32-trial pass are staged in shared
// memory ([trial][row], 64 KB) and written in natural row order: a trial's
// 256 keys are one coalesced 2 KB store, so the output layout and the
// generator order the stable grouping needs are unchanged.  Hub rows are
// left to hub_kernel (launched after, its stores win).
constexpr int kWin = 256;                      // rows per window = threads per CTA
constexpr int kWT = 16;                        // trials per staged pass (32 KB of keys)

template <int S, int L, bool PAD>
__device__ __forceinline__ uint64_t row_key(const uint32_t (&v)[8], uint32_t A, uint32_t B,
                                            uint64_t seed, int j);

template <int S, int L, bool PAD>
__device__ __forceinline__ void win_short(const uint32_t *sA, const uint32_t *sB, const uint32_t (&v)[8],
                                          uint64_t *sK, int lr, bool act, int tp0, int T, uint64_t seed,
                                          int t0) {
  for (int j = 0; j < T; ++j) {
    const uint64_t key = row_key<S, L, PAD>(v, sA[tp0 + j], sB[tp0 + j], seed, t0 + tp0 + j);
    if (act) sK[j * kWin + lr] = key;
  }
}

template <int S>
__global__ void __launch_bounds__(kWin, 4) minhash_win_kernel(const __grid_constant__ MinhashArgs a) {
  extern __shared__ __align__(16) unsigned char smraw[];
  uint64_t *sK = reinterpret_cast<uint64_t *>(smraw);                 // [kWT][kWin]
  uint32_t *sA = reinterpret_cast<uint32_t *>(sK + kWT * kWin);
  uint32_t *sB = sA + a.nt;
  __shared__ uint16_t sOrd[kWin];
  __shared__ uint32_t sCnt[12], sCur[12], sLong;
  __shared__ int64_t sWin;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, t = threadIdx.x;
  for (int i = t; i < a.nt; i += kWin) {
    sA[i] = a.A[a.t0 + i];
    sB[i] = a.B[a.t0 + i];
  }
  const int64_t nwin = (a.nrows + kWin - 1) / kWin;
  for (;;) {
    if (t == 0) sWin = (int64_t)atomicAdd(a.counter, 1ull);
    if (t < 12) sCnt[t] = 0;
    __syncthreads();
    const int64_t win = sWin;
    if (win >= nwin) break;
    const int64_t r0 = win * kWin;
    const int64_t r = r0 + t;
    const int len = r < a.nrows ? a.rlen[r] : 0;
    // class: 1..8 short (register rows), 9 long (lane = trial), 10 hub / none
    const int cls = len == 0 ? 10 : len <= 8 ? len : len <= kHubLen ? 9 : 10;
    atomicAdd(&sCnt[cls], 1u);
    __syncthreads();
    if (t == 0) {
      uint32_t run = 0;
      for (int c = 0; c < 12; ++c) {
        sCur[c] = run;
        run += sCnt[c];
      }
      sLong = 0;
    }
    __syncthreads();
    sOrd[atomicAdd(&sCur[cls], 1u)] = (uint16_t)t;
    __syncthreads();
    const int nshort = (int)(sCnt[1] + sCnt[2] + sCnt[3] + sCnt[4] + sCnt[5] + sCnt[6] + sCnt[7] + sCnt[8]);
    const int nlong = (int)sCnt[9];
    // this lane's short row, in registers for every pass
    const int slot = w * 32 + lane;
    const bool act = slot < nshort;
    const int lr = act ? sOrd[slot] : 0;
    int rl = 0;
    uint32_t v[8];
    if (act) {
      rl = a.rlen[r0 + lr];
      const uint32_t *src = a.entries + a.rstart[r0 + lr];
#pragma unroll
      for (int e = 0; e < 8; ++e) v[e] = e < rl ? src[e] : 0xFFFFFFFFu;
    } else {
#pragma unroll
      for (int e = 0; e < 8; ++e) v[e] = 0xFFFFFFFFu;
    }
    const bool any_short = __any_sync(0xffffffffu, act);
    const int lw = __reduce_max_sync(0xffffffffu, (unsigned)rl);
    const int lmin = __reduce_min_sync(0xffffffffu, act ? (unsigned)rl : 8u);
    for (int tp0 = 0; tp0 < a.nt; tp0 += kWT) {
      const int T = min(kWT, a.nt - tp0);
      if (any_short) {
        // the warp's longest row sets the unrolled length; only a warp that
        // mixes lengths (a class boundary of the window order) pays the pad test
#define SG_WS(L)                                                                          \
  case L:                                                                                 \
    if (lmin != lw) win_short<S, L, true>(sA, sB, v, sK, lr, act, tp0, T, a.seed, a.t0);  \
    else win_short<S, L, false>(sA, sB, v, sK, lr, act, tp0, T, a.seed, a.t0);            \
    break;
        switch (lw) {
          SG_WS(1) SG_WS(2) SG_WS(3) SG_WS(4) SG_WS(5) SG_WS(6) SG_WS(7)
          default: SG_WS(8)
        }
#undef SG_WS
      }
      // long rows, one per warp at a time (dynamic), lane = trial
      for (;;) {
        int li = 0;
        if (lane == 0) li = (int)atomicAdd(&sLong, 1u);
        li = __shfl_sync(0xffffffffu, li, 0);
        if (li >= nlong) break;
        const int lrow = sOrd[nshort + li];
        const int ll = a.rlen[r0 + lrow];
        const uint32_t *src = a.entries + a.rstart[r0 + lrow];
        // lanes = (trial tl, entry part): 32 / kWT parts scan interleaved
        // entries, merged by shuffles
        constexpr int NP = 32 / kWT;
        const int tl = lane & (kWT - 1), part = lane / kWT;
        const int j = tp0 + (tl < T ? tl : 0);
        const uint32_t A = sA[j], B = sB[j];
        uint32_t m[S];
#pragma unroll
        for (int i = 0; i < S; ++i) m[i] = 0xFFFFFFFFu;
        int e = part;
        for (; e + 3 * NP < ll; e += 4 * NP) {
          const uint32_t x0 = src[e], x1 = src[e + NP], x2 = src[e + 2 * NP], x3 = src[e + 3 * NP];
          insert_min<S>(m, m31_hash(A, B, x0));
          insert_min<S>(m, m31_hash(A, B, x1));
          insert_min<S>(m, m31_hash(A, B, x2));
          insert_min<S>(m, m31_hash(A, B, x3));
        }
        for (; e < ll; e += NP) insert_min<S>(m, m31_hash(A, B, src[e]));
        for (int o = kWT; o < 32; o <<= 1) {
          uint32_t x[S];
#pragma unroll
          for (int i = 0; i < S; ++i) x[i] = __shfl_xor_sync(0xffffffffu, m[i], o);
#pragma unroll
          for (int i = 0; i < S; ++i) insert_min<S>(m, x[i]);
        }
        if (part == 0 && tl < T) sK[tl * kWin + lrow] = fmix(shingle_id<S>(m, a.seed, a.t0 + j));
      }
      __syncthreads();
      // natural-order write-out: trial j's kWin keys are contiguous
      const int nr = (int)min((int64_t)kWin, a.nrows - r0);
      for (int j = 0; j < T; ++j) {
        if (t < nr) a.keys[(int64_t)(tp0 + j) * a.key_stride + r0 + t] = sK[j * kWin + t];
      }
      if (a.kbin) {
        for (int idx = t; idx < T * (kWin / 4); idx += kWin) {
          const int j = idx / (kWin / 4), q = idx % (kWin / 4);
          if (4 * q < nr) {
            const uint32_t *hi = reinterpret_cast<const uint32_t *>(sK + j * kWin + 4 * q);
            const uint32_t word = (hi[1] >> 24) | ((hi[3] >> 24) << 8) | ((hi[5] >> 24) << 16) |
                                  ((hi[7] >> 24) << 24);
            *reinterpret_cast<uint32_t *>(a.kbin + (int64_t)(tp0 + j) * a.key_stride + r0 + 4 * q) = word;
          }
        }
      }
      __syncthreads();
      if (t == 0) sLong = 0;
      __syncthreads();
    }
  }
}

template <int S>
cudaError_t launch_win(MhParams &P, int num_sms, cudaStream_t st) {
  const size_t smem = (size_t)kWT * kWin * 8 + (size_t)2 * P.a.nt * 4;
  auto kern = minhash_win_kernel<S>;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  int per_sm = 0;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, kWin, smem);
  if (e != cudaSuccess) return e;
  per_sm = std::max(per_sm, 1);
  const int64_t nwin = (P.a.nrows + kWin - 1) / kWin;
  const int grid = (int)std::min<int64_t>((int64_t)num_sms * per_sm, std::max<int64_t>(nwin, 1));
  kern<<<grid, kWin, smem, st>>>(P.a);
  ++g_launches;
  if ((e = cudaGetLastError()) != cudaSuccess) return e;
  const size_t hsm = (size_t)kHubStage * 4;
  if ((e = cudaFuncSetAttribute(hub_kernel<S>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                (int)hsm)) != cudaSuccess)
    return e;
  hub_kernel<S><<<num_sms * 3, kMhThreads, hsm, st>>>(P);
  ++g_launches;
  return cudaGetLastError();
}

// Short rows (pass II) take 16-row tiles: a trial's keys of one tile are a
// full 128 B line; long rows (pass I) keep 8-row tiles (the stage holds them).
// SG_MH_WIN=1 (A/B): the windowed row-per-lane kernel instead of the 16-row
// tile kernel for pass II (parity-green, measured slower on gos2m: hash2 49.9
// vs 43.9 ms; ncu: 11.1e9 vs 10.9e9 warp-instructions per 64-trial chunk —
// the per-(row, trial) key mixing, staging and the long rows' lane = trial
// scans cost as much as the tile kernel's row overheads).
static bool use_tile16() {
  static const bool v = [] {
    const char *e = getenv("SG_MH_WIN");
    return !(e && atoi(e) != 0);
  }();
  return v;
}

template <int S>
cudaError_t launch_s(MhParams &P, int num_sms, cudaStream_t st) {
  if (P.a.tile_rows == 16) return use_tile16() ? launch_tile<S, 16>(P, num_sms, st) : launch_win<S>(P, num_sms, st);
  return launch_tile<S, 8>(P, num_sms, st);
}

// ---- short rows, lane = row (pass II) ----------------------------------------
// Pass-II rows are the member lists of first-level shingles: ~5 entries on
// the GOS-shaped graph.  Rows of 2..8 entries are laid out by length class
// (row_classes below) and taken 32 at a time by a warp, one row per lane: the
// row sits in registers, every trial's (A, B) is a shared-memory broadcast,
// and the 32 keys of a trial are one coalesced 256 B store.  A warp's rows
// share their length except at the few class boundaries, so the predicated
// 8-entry loop does not diverge.
constexpr int kShortMax = 8;

// One trial of a row held in registers: v[0, L) (L compile-time: no
// predicated slots when the whole warp shares the length).
template <int S, int L, bool PAD>
__device__ __forceinline__ uint64_t row_key(const uint32_t (&v)[kShortMax], uint32_t A, uint32_t B,
                                            uint64_t seed, int j) {
  uint32_t m[S];
#pragma unroll
  for (int i = 0; i < S; ++i) m[i] = 0xFFFFFFFFu;
#pragma unroll
  for (int e = 0; e < L; ++e) insert_min<S>(m, PAD ? hash_or_pad(A, B, v[e]) : m31_hash(A, B, v[e]));
  return fmix(shingle_id<S>(m, seed, j));
}

template <int S, int L, bool PAD = false>
__device__ __forceinline__ void rows_trials(const MinhashArgs &a, const uint32_t *sA, const uint32_t *sB,
                                            const uint32_t (&v)[kShortMax], int64_t r, bool valid) {
  uint64_t *dst = a.keys + r;
  for (int j = 0; j < a.nt; ++j) {
    const uint64_t key = row_key<S, L, PAD>(v, sA[j], sB[j], a.seed, a.t0 + j);
    if (valid) dst[(int64_t)j * a.key_stride] = key;
  }
}

template <int S>
__global__ void __launch_bounds__(256) minhash_rows_kernel(const __grid_constant__ MinhashArgs a) {
  extern __shared__ uint32_t sAB[];
  uint32_t *sA = sAB, *sB = sAB + a.nt;
  for (int i = threadIdx.x; i < a.nt; i += blockDim.x) {
    sA[i] = a.A[a.t0 + i];
    sB[i] = a.B[a.t0 + i];
  }
  __syncthreads();
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const int lane = threadIdx.x & 31;
  for (int64_t w0 = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; w0 * 32 < a.nrows; w0 += nw) {
    const int64_t r = w0 * 32 + lane;
    const bool valid = r < a.nrows;
    int len = 0;
    uint32_t v[kShortMax];
    if (valid) {
      len = a.rlen[r];
      const uint32_t *src = a.entries + a.rstart[r];
#pragma unroll
      for (int e = 0; e < kShortMax; ++e) v[e] = e < len ? src[e] : 0xFFFFFFFFu;
    } else {
#pragma unroll
      for (int e = 0; e < kShortMax; ++e) v[e] = 0xFFFFFFFFu;
    }
    // rows are laid out by length class: the warp almost always shares one
    // length (compile-time unrolled, no idle slots); at a class boundary the
    // longest length is used, the padding (all-ones) never among the minima
    const int lw = __reduce_max_sync(0xffffffffu, (unsigned)len);
    const int lmin = __reduce_min_sync(0xffffffffu, (unsigned)len);
    if (lmin != lw) {                          // class boundary / last rows: padded slots
      rows_trials<S, kShortMax, true>(a, sA, sB, v, r, valid);
      continue;
    }
    switch (lw) {
      case 1: rows_trials<S, 1>(a, sA, sB, v, r, valid); break;
      case 2: rows_trials<S, 2>(a, sA, sB, v, r, valid); break;
      case 3: rows_trials<S, 3>(a, sA, sB, v, r, valid); break;
      case 4: rows_trials<S, 4>(a, sA, sB, v, r, valid); break;
      case 5: rows_trials<S, 5>(a, sA, sB, v, r, valid); break;
      case 6: rows_trials<S, 6>(a, sA, sB, v, r, valid); break;
      case 7: rows_trials<S, 7>(a, sA, sB, v, r, valid); break;
      default: rows_trials<S, 8>(a, sA, sB, v, r, valid); break;
    }
  }
}

template <int S>
cudaError_t launch_rows(const MinhashArgs &a, int num_sms, cudaStream_t st) {
  const int64_t warps = (a.nrows + 31) / 32;
  const int grid = (int)std::min<int64_t>((warps + 7) / 8, (int64_t)num_sms * 8);
  minhash_rows_kernel<S><<<grid, 256, (size_t)a.nt * 8, st>>>(a);
  ++g_launches;
  return cudaGetLastError();
}

// ---- row classes: rows of 2..8 entries by length, then the longer ones --------
__global__ void row_class_hist_kernel(const int32_t *__restrict__ rlen, int64_t n, unsigned long long *cnt) {
  __shared__ unsigned int h[kShortMax + 2];
  if (threadIdx.x < kShortMax + 2) h[threadIdx.x] = 0;
  __syncthreads();
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    atomicAdd(&h[min(rlen[i], kShortMax + 1)], 1u);
  __syncthreads();
  if (threadIdx.x < kShortMax + 2 && h[threadIdx.x]) atomicAdd(&cnt[threadIdx.x], (unsigned long long)h[threadIdx.x]);
}

__global__ void row_class_scatter_kernel(const int64_t *__restrict__ rstart, const int32_t *__restrict__ rlen,
                                         int64_t n, unsigned long long *cursor, uint32_t *perm,
                                         int64_t *rstart_p, int32_t *rlen_p) {
  const int lane = threadIdx.x & 31;
  const uint32_t lt = (1u << lane) - 1u;
  for (int64_t i0 = ((int64_t)blockIdx.x * blockDim.x) & ~31ll; i0 < n; i0 += (int64_t)gridDim.x * blockDim.x) {
    const int64_t i = i0 + (threadIdx.x & ~31) + lane;
    const bool valid = i < n;
    const int len = valid ? rlen[i] : 0;
    const int cls = valid ? min(len, kShortMax + 1) : -1;
    const uint32_t peers = __match_any_sync(0xffffffffu, cls);
    const int leader = __ffs(peers) - 1;
    unsigned long long base = 0;
    if (valid && lane == leader) base = atomicAdd(&cursor[cls], (unsigned long long)__popc(peers));
    base = __shfl_sync(0xffffffffu, base, leader);
    if (valid) {
      const int64_t p = (int64_t)base + __popc(peers & lt);
      perm[p] = (uint32_t)i;
      rstart_p[p] = rstart[i];
      rlen_p[p] = len;
    }
  }
}

// ---- id recomputation for getters / report (one thread per request) --------
__global__ void shingle_ids_kernel(const int64_t *rstart, const int32_t *rlen,
                                   const uint32_t *entries, const uint32_t *A, const uint32_t *B,
                                   int s, uint64_t seed, const int64_t *req_row,
                                   const int32_t *req_trial, int64_t nreq, uint64_t *ids) {
  for (int64_t q = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; q < nreq;
       q += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = req_row[q];
    const int j = req_trial[q];
    const uint32_t *row = entries + rstart[r];
    const int len = rlen[r];
    uint32_t m[kMaxS];
    for (int i = 0; i < kMaxS; ++i) m[i] = 0xFFFFFFFFu;
    for (int e = 0; e < len; ++e) {
      uint32_t h = m31_hash(A[j], B[j], row[e]);
      if (h >= m[s - 1]) continue;
      int i = s - 1;
      while (i > 0 && m[i - 1] > h) {
        m[i] = m[i - 1];
        --i;
      }
      m[i] = h;
    }
    uint64_t id;
    if (s == 1) {
      id = m[0];
    } else if (s == 2) {
      id = ((uint64_t)m[0] << 31) | m[1];
    } else {
      uint64_t z = fmix(seed ^ fmix((uint64_t)j + 1));
      for (int i = 0; i < s; ++i) z = fmix(z + (uint64_t)m[i]);
      id = z;
    }
    ids[q] = id;
  }
}

}  // namespace

cudaError_t minhash(const MinhashArgs &a, int num_sms, cudaStream_t st) {
  if (a.nrows == 0 || a.nt == 0) return cudaSuccess;
  if (a.key_stride % kRowTile != 0 || (a.tile_rows != 8 && a.tile_rows != 16))
    return cudaErrorInvalidValue;
  MhParams P;
  P.a = a;
  // trial passes: full groups of 32 lanes (one trial per lane), then the
  // binary digits of nt mod 32 (2^b trials x 32/2^b neighbour parts)
  int np = 0, t = 0;
  while (a.nt - t >= 32) {
    P.pass[np++] = TrialPass{(int16_t)t, 5, 0};
    t += 32;
  }
  for (int b = 4; b >= 0; --b) {
    if ((a.nt - t) & (1 << b)) {
      P.pass[np++] = TrialPass{(int16_t)t, (int8_t)b, (int8_t)(5 - b)};
      t += 1 << b;
    }
  }
  P.npass = np;
  switch (a.s) {
    case 1: return launch_s<1>(P, num_sms, st);
    case 2: return launch_s<2>(P, num_sms, st);
    case 3: return launch_s<3>(P, num_sms, st);
    case 4: return launch_s<4>(P, num_sms, st);
    case 5: return launch_s<5>(P, num_sms, st);
    case 6: return launch_s<6>(P, num_sms, st);
    case 7: return launch_s<7>(P, num_sms, st);
    case 8: return launch_s<8>(P, num_sms, st);
    default: return cudaErrorInvalidValue;
  }
}

cudaError_t minhash_short_rows(const MinhashArgs &a, int num_sms, cudaStream_t st) {
  if (a.nrows == 0 || a.nt == 0) return cudaSuccess;
  switch (a.s) {
    case 1: return launch_rows<1>(a, num_sms, st);
    case 2: return launch_rows<2>(a, num_sms, st);
    case 3: return launch_rows<3>(a, num_sms, st);
    case 4: return launch_rows<4>(a, num_sms, st);
    case 5: return launch_rows<5>(a, num_sms, st);
    case 6: return launch_rows<6>(a, num_sms, st);
    case 7: return launch_rows<7>(a, num_sms, st);
    case 8: return launch_rows<8>(a, num_sms, st);
    default: return cudaErrorInvalidValue;
  }
}

int32_t short_row_max() { return kShortMax; }

cudaError_t row_classes(const int64_t *rstart, const int32_t *rlen, int64_t n, unsigned long long *d_cnt,
                        unsigned long long *d_cursor, const unsigned long long *h_start, uint32_t *perm,
                        int64_t *rstart_p, int32_t *rlen_p, cudaStream_t st) {
  if (n == 0) return cudaSuccess;
  const int grid = (int)std::min<int64_t>((n + 255) / 256, 148 * 8);
  if (!h_start) {
    cudaError_t e = cudaMemsetAsync(d_cnt, 0, (kShortMax + 2) * 8, st);
    if (e != cudaSuccess) return e;
    row_class_hist_kernel<<<grid, 256, 0, st>>>(rlen, n, d_cnt);
    ++g_launches;
    return cudaGetLastError();
  }
  cudaError_t e = cudaMemcpyAsync(d_cursor, h_start, (kShortMax + 2) * 8, cudaMemcpyHostToDevice, st);
  if (e != cudaSuccess) return e;
  row_class_scatter_kernel<<<grid, 256, 0, st>>>(rstart, rlen, n, d_cursor, perm, rstart_p, rlen_p);
  ++g_launches;
  return cudaGetLastError();
}

cudaError_t shingle_ids(const int64_t *rstart, const int32_t *rlen, const uint32_t *entries,
                        const uint32_t *A, const uint32_t *B, int32_t s, uint64_t seed,
                        const int64_t *req_row, const int32_t *req_trial, int64_t nreq,
                        uint64_t *ids, cudaStream_t st) {
  if (nreq == 0) return cudaSuccess;
  const int grid = (int)std::min<int64_t>((nreq + 255) / 256, 148 * 16);
  shingle_ids_kernel<<<grid, 256, 0, st>>>(rstart, rlen, entries, A, B, s, seed, req_row,
                                           req_trial, nreq, ids);
  return cudaGetLastError();
}

}  // namespace sg
