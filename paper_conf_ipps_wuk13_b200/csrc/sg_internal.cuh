// sg_internal.cuh — internal definitions of libshingle (B200 / sm_100a).
//
// Product code: shares nothing with oracle/ (test infrastructure).  All
// arithmetic here is restated from the paper and DESIGN.md's readings.
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <string>
#include <utility>
#include <vector>

#include "../../include/shingle.h"

namespace sg {

// P = 2^31 - 1, "a big prime number" (AMB-1).
constexpr uint32_t kP = 0x7FFFFFFFu;
constexpr int kMaxS = 8;        // s bound of the ABI
constexpr int kMaxC = 1024;     // c bound of the ABI

// ----------------------------------------------------------------------------
// 64-bit mixing: the splitmix64 finaliser and its inverse (bijection on 2^64).
// Used for (a) the hash-pair stream (AMB-2), (b) the s >= 3 shingle fold
// (AMB-4), (c) the grouping key key = fmix(id) (AMB-19).
// ----------------------------------------------------------------------------
__host__ __device__ __forceinline__ uint64_t fmix(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ull;
  z = (z ^ (z >> 27)) * 0x94d049bb133111ebull;
  return z ^ (z >> 31);
}

__host__ __device__ __forceinline__ uint64_t unxorshift(uint64_t z, int s) {
  uint64_t x = z;
  for (int i = 0; i < 64 / s + 1; ++i) x = z ^ (x >> s);
  return x;
}

__host__ __device__ __forceinline__ uint64_t fmix_inv(uint64_t z) {
  z = unxorshift(z, 31);
  z *= 0x319642b2d24d8ec3ull;   // inverse of 0x94d049bb133111eb mod 2^64
  z = unxorshift(z, 27);
  z *= 0x96de1b173f119089ull;   // inverse of 0xbf58476d1ce4e5b9 mod 2^64
  return unxorshift(z, 30);
}

// (A*v + B) mod (2^31 - 1) with one 32x32->64 multiply-add and a Mersenne
// fold: t < 2^62, x = (t & P) + (t >> 31) < 2P (t <= (P-1)P), so one
// conditional subtract finishes.  The unsigned min picks x or x - P.
__device__ __forceinline__ uint32_t m31_hash(uint32_t A, uint32_t B, uint32_t v) {
  uint64_t t = (uint64_t)A * v + B;
  uint32_t lo = (uint32_t)t & kP;
  uint32_t hi = (uint32_t)(t >> 31);
  uint32_t x = lo + hi;
  uint32_t y = x - kP;
  return x < y ? x : y;
}

// ----------------------------------------------------------------------------
// Handle
// ----------------------------------------------------------------------------
enum State : int32_t {
  kEmpty = -1,    // a shingle_graph_load failed: no valid graph resident
  kCreated = 0,   // CSR resident
  kPassed1 = 1,   // pass I rows selected (keys computed unless deferred)
  kGrouped1 = 2,  // G_I resident
  kPassed2 = 3,   // pass II rows selected
  kGrouped2 = 4,  // G_II resident
  kPoisoned = 99
};

// Device buffer owned by the handle (stream-ordered pool allocations).
struct DBuf {
  void *p = nullptr;
  size_t bytes = 0;
};

// Keys of a contiguous range of trials [t0, t0 + nt): uint64 [nt][key_stride].
struct KeyChunk {
  int32_t t0 = 0, nt = 0;
  bool computed = false;
  DBuf keys;
  DBuf kbin;                       // top key bytes (single rank, grouping v1), or empty
  DBuf ctr;                        // the min-hash tile counters (kept while in flight)
  cudaEvent_t done = nullptr;      // recorded on the side stream when computed there
};

// One shingling pass on this rank.
struct PassOut {
  int32_t s = 0, c = 0;
  uint64_t seed = 0;
  int64_t nrows = 0;            // local rows with >= s entries
  int64_t key_stride = 0;       // nrows rounded up to the row tile
  std::vector<uint32_t> hA, hB; // hash pairs (host copy)
  DBuf A, B;                    // uint32 [c]
  DBuf rstart;                  // int64 [nrows] first entry of each row
  DBuf rlen;                    // int32 [nrows]
  DBuf rowid;                   // uint32 [nrows] generator value (pass I: vertex id)
  const uint32_t *entries = nullptr;  // row entries (pass I: col; pass II: G_I members)
  std::vector<KeyChunk> chunks; // trial chunks sized to the free HBM
  bool deferred = false;        // keys computed chunk by chunk inside group_by_shingle
  bool kbin = false;            // the min-hash kernels also write the keys' top bytes
  std::vector<int64_t> blocks;  // row blocks in generator order (multi-rank exchange pieces)
  // pass II, one rank: key positions in length-class order;
  // key position i belongs to row perm[i]; positions [0, n_split) are rows of
  // <= 8 entries (one row per lane), the rest take the tile / hub kernels
  DBuf perm;                    // uint32 [nrows] (empty: identity)
  DBuf rstart_p, rlen_p;        // rstart / rlen in key-position order
  int64_t n_split = 0;
};

// Grouped pairs of one level on this rank: per-trial segments of `members`
// in canonical (trial, key, member) order with one head bit per group start.
struct Groups {
  int32_t c = 0;
  int64_t npairs = 0;
  std::vector<int64_t> seg;            // [c+1] pair offsets per trial (host)
  DBuf members;                        // uint32 [npairs]
  DBuf head;                           // uint32 [(npairs + 31) / 32] head bits
  DBuf okeys;                          // uint64 [npairs] sorted keys (multi-rank only)
};

constexpr int kNumStages = 19;
enum StageId {
  kStPass1 = 0, kStGroup1 = 1, kStPass2 = 2, kStGroup2 = 3,
  kStSelect1 = 4, kStHash1 = 5, kStSelect2 = 6, kStHash2 = 7,
  kStHist1 = 8, kStScatter1 = 9, kStLocal1 = 10,
  kStHist2 = 11, kStScatter2 = 12, kStLocal2 = 13,
  kStX1 = 14, kStX2 = 15,
  kStFine1 = 16, kStFine2 = 17,    // second-level (fine) split of two-level plans
  kStReport = 18                   // Phase III on the device (outside the metric)
};

struct Exchange;  // multi-GPU (exchange.cu)

// Error propagation inside the library: thrown by fail(), caught at the ABI.
struct Fail {
  sg_status st;
};
[[noreturn]] void fail(sg_graph *g, sg_status st, const std::string &m);
void ck(sg_graph *g, cudaError_t e, const char *what);

}  // namespace sg

struct sg_graph {
  int32_t state = sg::kCreated;
  sg_status poison = SG_OK;
  std::string err;
  int32_t device = 0;
  cudaStream_t stream = nullptr;
  bool own_stream = false;
  cudaStream_t side = nullptr;     // min-hash of later trial chunks, overlapped with grouping
  int32_t rank = 0, world = 1;
  sg::Exchange *xch = nullptr;      // owner-routed exchange path (world > 1, or SG_DIST_EXCHANGE)
  bool peer_xch = false;            // SG_DIST_PEER: fused exchange over peer memory
  cudaMemPool_t pool = nullptr;     // the handle's private stream-ordered pool
  int num_sms = 148;
  // graph (global n; this rank's rows [row_lo, row_hi))
  int64_t n = 0, nnz_global = 0;
  int64_t row_lo = 0, row_hi = 0;
  int64_t nnz_local = 0;
  sg::DBuf row_ptr;   // int64 [rows + 1], rebased to 0
  sg::DBuf col;       // uint32 [nnz_local] (empty with SG_HOST_CSR)
  const uint32_t *col_dev = nullptr;   // the entries as the kernels read them: col.p, or the
                                       // device alias of the caller's mapped host array
  void *col_reg = nullptr;             // host range this handle registered (SG_HOST_CSR)
  // passes and groups
  sg::PassOut pass[2];
  sg::Groups grp[2];
  // global counts (summed over ranks)
  int64_t n_e_global = 0, s1p_global = 0, s1p_k0 = 0;
  int64_t groups_global[2] = {0, 0};
  int64_t pairs_global[2] = {0, 0};
  int64_t e2_global = -1;       // pass-II entries (sum of |L| over S1'), lazily
  long long launch_base = 0;    // g_launches at create / reset
  // report_overlapping_clusters two-call pattern: the sizing call keeps its
  // result here for the filling call (same mode / min_size); cleared by it
  // and by reset
  bool ov_valid = false;
  int32_t ov_mode = 0, ov_min = 0;
  std::vector<int64_t> ov_offs;
  std::vector<uint32_t> ov_verts;
  // stage timing: event pairs per stage (a stage may span several chunks)
  std::vector<cudaEvent_t> ev_pool;
  size_t ev_next = 0;
  std::vector<std::pair<int, int>> st[sg::kNumStages];
  int64_t mem_budget = 0;       // test hook: cap on planned bytes (0 = free HBM)
  int64_t bytes_live = 0;       // device bytes currently held by this handle
  // plan_pass memo per level: the device memory query (cudaMemGetInfo) can
  // take milliseconds under load, and repeated steps plan the same pass in
  // the same allocation state
  struct PlanMemo {
    int64_t nrows = -1, c = -1, live = -1, cached = -1;
    bool deferred = false, kbin = false;
    std::vector<std::pair<int32_t, int32_t>> chunks;
  } plan_memo[2];
  std::vector<sg::DBuf> cache;  // freed blocks kept for reuse (best fit)
  int64_t bytes_cached = 0;
  // allocation diagnostics since the last reset (SG_ALLOC_LOG prints them)
  int64_t n_pool_allocs = 0, n_cache_releases = 0, n_trims = 0;
  double alloc_host_ms = 0;
};
