// api.cu — the C ABI of libshingle (include/shingle.h): handle lifecycle,
// stage sequencing, HBM planning, timing and getters.  Every step of the hot
// path runs in the kernels of kernels_{pass,minhash,group}.cu; there is no
// CPU fallback.
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <memory>
#include <string>
#include <vector>

#include <nvtx3/nvToolsExt.h>

#include "exchange.h"
#include "kernels.h"
#include "report.h"
#include "sg_internal.cuh"

using namespace sg;

namespace {
thread_local std::string t_err;

void set_err(sg_graph *g, const std::string &m) {
  if (g) g->err = m;
  t_err = m;
}
}  // namespace

namespace sg {
[[noreturn]] void fail(sg_graph *g, sg_status st, const std::string &m) {
  set_err(g, m);
  if (g && (st == SG_ECUDA || st == SG_ENCCL)) {
    g->poison = st;
    g->state = kPoisoned;
  }
  throw Fail{st};
}

void ck(sg_graph *g, cudaError_t e, const char *what) {
  if (e != cudaSuccess) fail(g, SG_ECUDA, std::string(what) + ": " + cudaGetErrorString(e));
}
}  // namespace sg

namespace {

#define CK(call) ck(g, (call), #call)

// Per-handle buffer cache: freed buffers are kept and handed out again by
// best fit, so repeated runs (bench steps, resets) allocate nothing and the
// stream-ordered pool does not fragment and grow.
// SG_NO_CACHE=1 (A/B hook): freed buffers go straight back to the handle's
// stream-ordered pool (which keeps them reserved for reuse).
bool no_cache() {
  static const bool v = getenv("SG_NO_CACHE") != nullptr;
  return v;
}

// Blocks above SG_CACHE_MAX_BYTES (default: no limit) go straight back to
// the stream-ordered pool instead of the handle's best-fit cache.
size_t cache_max_bytes() {
  static const size_t v = [] {
    const char *e = getenv("SG_CACHE_MAX_BYTES");
    return e ? (size_t)atoll(e) : (size_t)-1;
  }();
  return v;
}

void cache_put(sg_graph *g, void *p, size_t bytes) {
  if (no_cache() || bytes > cache_max_bytes()) {
    cudaFreeAsync(p, g->stream);
    return;
  }
  g->cache.push_back({p, bytes});
  g->bytes_cached += (int64_t)bytes;
}

void cache_release(sg_graph *g) {
  for (auto &c : g->cache) cudaFreeAsync(c.p, g->stream);
  g->cache.clear();
  g->bytes_cached = 0;
}

void *cache_take(sg_graph *g, size_t bytes, size_t *got) {
  size_t best = g->cache.size();
  for (size_t i = 0; i < g->cache.size(); ++i) {
    const size_t b = g->cache[i].bytes;
    if (b >= bytes && b <= bytes + bytes / 4 + (1u << 20) &&
        (best == g->cache.size() || b < g->cache[best].bytes))
      best = i;
  }
  if (best == g->cache.size()) return nullptr;
  void *p = g->cache[best].p;
  *got = g->cache[best].bytes;
  g->bytes_cached -= (int64_t)*got;
  g->cache.erase(g->cache.begin() + (long)best);
  return p;
}

void dfree(sg_graph *g, DBuf &b);

void dalloc(sg_graph *g, DBuf &b, size_t bytes) {
  if (b.p) dfree(g, b);
  if (bytes == 0) bytes = 16;
  bytes = (bytes + 255) & ~(size_t)255;
  size_t got = 0;
  if (void *c = cache_take(g, bytes, &got)) {
    b.p = c;
    b.bytes = got;
    g->bytes_live += (int64_t)got;
    return;
  }
  void *p = nullptr;
  const auto t0 = std::chrono::steady_clock::now();
  ++g->n_pool_allocs;
  cudaError_t e = cudaMallocFromPoolAsync(&p, bytes, g->pool, g->stream);
  if (e != cudaSuccess) {
    // the device is full: return every cached block to the pool and retry
    // (handing blocks back one at a time, largest first, was measured to
    // leave the 640M-edge config in a pathological state: 12.8 s per step)
    cudaGetLastError();
    ++g->n_cache_releases;
    cache_release(g);
    e = cudaMallocFromPoolAsync(&p, bytes, g->pool, g->stream);
  }
  if (e != cudaSuccess) {
    // the pool's free blocks may be too fragmented for one large request
    // (e.g. after a step with another (s, c)): return them to the device and
    // map the request afresh (the handle's private pool only)
    cudaGetLastError();
    ++g->n_trims;
    cudaStreamSynchronize(g->stream);
    cudaMemPoolTrimTo(g->pool, 0);
    e = cudaMallocFromPoolAsync(&p, bytes, g->pool, g->stream);
  }
  g->alloc_host_ms += std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
  if (e != cudaSuccess) {
    cudaGetLastError();
    size_t fr = 0, tot = 0;
    cudaMemGetInfo(&fr, &tot);
    cudaGetLastError();
    char buf[192];
    snprintf(buf, sizeof buf, "device allocation of %zu bytes failed (device free %zu of %zu bytes)",
             bytes, fr, tot);
    fail(g, SG_ENOMEM, buf);
  }
  b.p = p;
  b.bytes = bytes;
  g->bytes_live += (int64_t)bytes;
}

void dfree(sg_graph *g, DBuf &b) {
  if (b.p) {
    cache_put(g, b.p, b.bytes);
    g->bytes_live -= (int64_t)b.bytes;
  }
  b.p = nullptr;
  b.bytes = 0;
}

template <typename T>
T *ptr(const DBuf &b) {
  return reinterpret_cast<T *>(b.p);
}

void sync(sg_graph *g) { CK(cudaStreamSynchronize(g->stream)); }

// ---- stage timing: CUDA events on the handle's stream ------------------------
int ev_take(sg_graph *g) {
  if (g->ev_next == g->ev_pool.size()) {
    cudaEvent_t e;
    CK(cudaEventCreate(&e));
    g->ev_pool.push_back(e);
  }
  return (int)g->ev_next++;
}

// Stage names (NVTX ranges for a timeline profiler; sg_get_stage_ms order).
const char *const kStageName[kNumStages] = {
    "pass1", "group1", "pass2", "group2", "select1", "hash1", "select2", "hash2", "hist1",
    "scatter1", "local1", "hist2", "scatter2", "local2", "exchange1", "exchange2", "fine1",
    "fine2", "report"};

void st_begin(sg_graph *g, int id, cudaStream_t st = nullptr) {
  if (!st) nvtxRangePushA(kStageName[id]);     // host-side range (nested stages nest)
  const int e = ev_take(g);
  CK(cudaEventRecord(g->ev_pool[(size_t)e], st ? st : g->stream));
  g->st[id].push_back({e, -1});
}

void st_end(sg_graph *g, int id, cudaStream_t st = nullptr) {
  const int e = ev_take(g);
  CK(cudaEventRecord(g->ev_pool[(size_t)e], st ? st : g->stream));
  g->st[id].back().second = e;
  if (!st) nvtxRangePop();
}

void st_clear(sg_graph *g) {
  for (auto &v : g->st) v.clear();
  g->ev_next = 0;
}

// `collective` calls (pass, group) run exchange steps on world > 1: a rank
// that fails inside one breaks a loopback group so its peers return too.
template <typename F>
sg_status guarded(sg_graph *g, F &&f, bool collective = false) {
  if (!g) {
    t_err = "null handle";
    return SG_EINVAL;
  }
  sg_status st = SG_OK;
  if (g->state == kPoisoned) {
    st = g->poison;
  } else {
    try {
      int dev = -1;
      cudaGetDevice(&dev);
      if (dev != g->device) CK(cudaSetDevice(g->device));
      f();
    } catch (const Fail &x) {
      st = x.st;
    } catch (const std::bad_alloc &) {
      set_err(g, "host allocation failed");
      st = SG_ENOMEM;
    }
  }
  if (st != SG_OK && collective && g->xch) exchange_abort(g->xch);
  return st;
}

void free_pass(sg_graph *g, PassOut &p) {
  bool side = false;
  for (auto &ch : p.chunks) side |= ch.done != nullptr;
  if (side) cudaStreamSynchronize(g->side);       // chunks still in flight there
  for (DBuf *b : {&p.A, &p.B, &p.rstart, &p.rlen, &p.rowid, &p.perm, &p.rstart_p, &p.rlen_p}) dfree(g, *b);
  for (auto &ch : p.chunks) {
    dfree(g, ch.keys);
    dfree(g, ch.kbin);
    dfree(g, ch.ctr);
    if (ch.done) cudaEventDestroy(ch.done);
  }
  p = PassOut();
}

void free_groups(sg_graph *g, Groups &q) {
  dfree(g, q.members);
  dfree(g, q.head);
  dfree(g, q.okeys);
  q = Groups();
}

// ---------------------------------------------------------------- validation
// One warp per row (hub rows of tens of thousands of entries do not serialise
// on one thread): row bounds, ids in [0, n), strictly increasing entries.
__global__ void validate_kernel(const int64_t *rp, const int32_t *col, int64_t rows, int64_t nnz,
                                int64_t n, int *bad) {
  const int lane = threadIdx.x & 31;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t u = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; u < rows; u += nw) {
    const int64_t a = rp[u], b = rp[u + 1];
    if (b < a || a < 0 || b > nnz) {
      if (lane == 0) atomicExch(bad, 1);
      continue;
    }
    bool ok = true;
    for (int64_t e = a + lane; e < b; e += 32) {
      const int32_t v = col[e];
      ok &= v >= 0 && (int64_t)v < n && (e == a || v > col[e - 1]);
    }
    if (!__all_sync(0xffffffffu, ok) && lane == 0) atomicExch(bad, 1);
  }
}

__global__ void rebase_kernel(int64_t *rp, int64_t n1, int64_t base) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n1;
       i += (int64_t)gridDim.x * blockDim.x)
    rp[i] -= base;
}

// ---------------------------------------------------------------- HBM planning
// Bytes the handle may still allocate: free device memory + blocks cached by
// the stream-ordered pool, capped by the SG_MEM_BUDGET test hook.
// SG_DEBUG_HOST: host-side timeline of the pass/group calls on stderr
// (diagnostics for the host gaps inside the stage events).
struct HostMark {
  bool on = getenv("SG_DEBUG_HOST") != nullptr;
  std::chrono::steady_clock::time_point t0 = std::chrono::steady_clock::now();
  void operator()(const char *what) {
    if (!on) return;
    const auto t = std::chrono::steady_clock::now();
    fprintf(stderr, "[sg-host] %-24s %8.3f ms\n", what,
            std::chrono::duration<double, std::milli>(t - t0).count());
    t0 = t;
  }
};

int64_t avail_bytes(sg_graph *g) {
  size_t fr = 0, tot = 0;
  CK(cudaMemGetInfo(&fr, &tot));
  uint64_t reserved = 0, used = 0;
  CK(cudaMemPoolGetAttribute(g->pool, cudaMemPoolAttrReservedMemCurrent, &reserved));
  CK(cudaMemPoolGetAttribute(g->pool, cudaMemPoolAttrUsedMemCurrent, &used));
  int64_t a = (int64_t)fr + (int64_t)(reserved - used) + g->bytes_cached - ((int64_t)1 << 30);
  if (g->mem_budget > 0) a = std::min<int64_t>(a, g->mem_budget - g->bytes_live);
  if (getenv("SG_DEBUG_MEM"))
    fprintf(stderr, "[sg] free %zu total %zu pool reserved %llu used %llu cached %lld live %lld -> avail %lld\n",
            fr, tot, (unsigned long long)reserved, (unsigned long long)used,
            (long long)g->bytes_cached, (long long)g->bytes_live, (long long)a);
  return a;
}

// Split the c trials into chunks so that the pass's keys and the grouping's
// scratch fit in HBM (grouping is per trial, so chunking is exact, AMB-5).
// Eager: all keys computed by shingle_pass.  Deferred: group_by_shingle
// computes each chunk's keys right before grouping it.
double scratch_per_pair(int64_t maxseg);

void plan_pass_uncached(sg_graph *g, PassOut &P);

// Memoised plan: same level, rows, trials and allocation state as a previous
// step (single rank; multi-rank plans agree across ranks through a
// collective, so they are always recomputed).
void plan_pass(sg_graph *g, PassOut &P, int level) {
  auto &m = g->plan_memo[level];
  if (!g->xch && m.nrows == P.nrows && m.c == P.c && m.live == g->bytes_live &&
      m.cached == g->bytes_cached) {
    P.deferred = m.deferred;
    P.kbin = m.kbin;
    P.chunks.clear();
    for (auto &tc : m.chunks) {
      KeyChunk k;
      k.t0 = tc.first;
      k.nt = tc.second;
      P.chunks.push_back(k);
    }
    return;
  }
  m.live = g->bytes_live;
  m.cached = g->bytes_cached;
  plan_pass_uncached(g, P);
  m.nrows = P.nrows;
  m.c = P.c;
  m.deferred = P.deferred;
  m.kbin = P.kbin;
  m.chunks.clear();
  for (auto &k : P.chunks) m.chunks.push_back({k.t0, k.nt});
}

bool use_group_v1();

// The min-hash kernels may also write each key's top byte (the coarse bin)
// for the byte histogram: single rank, stable grouping, rows in generator
// order, and only when the plan leaves room for them (below).
bool kbin_eligible(const sg_graph *g, const PassOut &P) {
  return !g->xch && use_group_v1() && P.perm.p == nullptr && !getenv("SG_NO_KBIN");
}

// One plan for `kb` bytes per resident key: eager (all keys resident, the
// scratch of `per` trials beside them) or deferred (keys of one chunk).
struct Plan {
  bool deferred = false;
  int64_t per = 0, nch = 0;
};

Plan make_plan(sg_graph *g, const PassOut &P, double kb, double avail) {
  const int64_t nr = P.nrows, c = P.c;
  const double keys_t = kb * (double)P.key_stride;              // keys of one trial
  const double scr_t = scratch_per_pair(nr) * (double)nr + 65536.0 * 8;   // scratch per trial
  const double members = 4.125 * (double)nr * (double)c + (1 << 20);
  Plan pl;
  int64_t ct = (int64_t)((avail - members - keys_t * c) / scr_t);
  if (g->xch) {
    // multi-rank: all keys are kept until their exchange (eager), sorted keys
    // are kept for the getters, send + receive buffers per chunk; every rank
    // uses the same trial chunks (the exchange rounds must match)
    const double mr_t = scr_t + 24.0 * (double)nr + 8.0 * (double)nr;
    ct = (int64_t)((avail - members - keys_t * c) / mr_t);
    ct = exchange_min(g, std::max<int64_t>(ct, 0));
    if (ct < 1) fail(g, SG_ENOMEM, "multi-rank pass needs all keys resident; not enough HBM");
  } else if (ct < 1) {
    ct = (int64_t)((avail - members) / (keys_t + scr_t));
    pl.deferred = true;
    if (ct < 1) {
      char buf[160];
      snprintf(buf, sizeof buf, "pass needs more HBM than available (%.0f B for the members alone)",
               members);
      fail(g, SG_ENOMEM, buf);
    }
  }
  ct = std::min<int64_t>(ct, c);
  pl.nch = (c + ct - 1) / ct;
  pl.per = (c + pl.nch - 1) / pl.nch;
  // whole 32-trial groups per chunk: the min-hash runs 32 trials per lane
  // pass and a tail pass (c mod 32 trials) costs a full pass per row, so
  // e.g. 200 = 64+64+64+8 (7 passes) rather than 67+67+66 (11 passes)
  if (pl.per < c && pl.per >= 32) pl.per = pl.per / 32 * 32;
  pl.nch = (c + pl.per - 1) / pl.per;
  return pl;
}

void plan_pass_uncached(sg_graph *g, PassOut &P) {
  const int64_t nr = P.nrows, c = P.c;
  // headroom: the plan's buffers are carved from one stream-ordered pool, and
  // a plan that fills the device to the last gigabyte fragments it (the
  // allocations then fail, the pool is trimmed and re-mapped inside the timed
  // stages: measured 0.26-1.6 s group2 swings on hub2m); plan against 90 %
  // of the available bytes minus 4 GB
  const double raw = (double)avail_bytes(g);
  const double avail = g->mem_budget > 0 ? raw        // test hook: exact budget
                                         : 0.9 * raw - 4.0e9;
  Plan pl = make_plan(g, P, 8.0, avail);
  P.kbin = false;
  if (kbin_eligible(g, P)) {
    // The key bytes of the byte histogram (1 B per resident key): planned at
    // 9 B per key when that plan has no more chunks than the 8 B one; else
    // carried in the 8 B plan's headroom when the device still holds them;
    // else left out (measured: unplanned they over-committed the eager plan
    // of the s = 3, c = 400 sweep point, 2.7 s per step; planned, its
    // deferred 5-chunk plan runs in 0.64 s; planned at 9 B they split gos2m
    // into 7 trial chunks instead of 4, +8 ms, while the 4-chunk plan holds
    // them in its headroom)
    const Plan p9 = make_plan(g, P, 9.0, avail);
    if (p9.nch <= pl.nch) {
      pl = p9;
      P.kbin = true;
    } else {
      const double scr_t = scratch_per_pair(nr) * (double)nr + 65536.0 * 8;
      const double members = 4.125 * (double)nr * (double)c + (1 << 20);
      const double resident = pl.deferred ? (double)pl.per : (double)c;
      const double need = members + resident * 9.0 * (double)P.key_stride + (double)pl.per * scr_t;
      P.kbin = need <= (g->mem_budget > 0 ? raw : 0.97 * raw);
    }
  }
  P.deferred = pl.deferred;
  P.chunks.clear();
  for (int64_t t = 0; t < c; t += pl.per) {
    KeyChunk k;
    k.t0 = (int32_t)t;
    k.nt = (int32_t)std::min<int64_t>(pl.per, c - t);
    P.chunks.push_back(k);
  }
}

bool use_group_v1();

// Pass II on one rank: lay the key positions out by row length so that rows
// of <= 8 entries are processed one per lane (minhash_short_rows).  The
// grouping is independent of the order of the pairs (v3 sorts each bucket by
// (key, member)), and the value of key position i is perm[i] (the S1' index).
void build_row_classes(sg_graph *g, PassOut &P, int64_t nrows) {
  const int NC = short_row_max() + 2;
  DBuf cnt, cur;
  dalloc(g, cnt, (size_t)NC * 8);
  dalloc(g, cur, (size_t)NC * 8);
  CK(row_classes(ptr<int64_t>(P.rstart), ptr<int32_t>(P.rlen), nrows, ptr<unsigned long long>(cnt),
                 nullptr, nullptr, nullptr, nullptr, nullptr, g->stream));
  std::vector<unsigned long long> h((size_t)NC);
  CK(cudaMemcpyAsync(h.data(), cnt.p, (size_t)NC * 8, cudaMemcpyDeviceToHost, g->stream));
  sync(g);
  std::vector<unsigned long long> start((size_t)NC, 0);
  unsigned long long run = 0;
  for (int c = 0; c < NC; ++c) {
    start[(size_t)c] = run;
    run += h[(size_t)c];
  }
  const int64_t n_short = (int64_t)start[(size_t)NC - 1];   // rows of <= 8 entries
  dalloc(g, P.perm, (size_t)nrows * 4);
  dalloc(g, P.rstart_p, (size_t)nrows * 8);
  dalloc(g, P.rlen_p, (size_t)nrows * 4);
  CK(row_classes(ptr<int64_t>(P.rstart), ptr<int32_t>(P.rlen), nrows, nullptr, ptr<unsigned long long>(cur),
                 start.data(), ptr<uint32_t>(P.perm), ptr<int64_t>(P.rstart_p), ptr<int32_t>(P.rlen_p),
                 g->stream));
  sync(g);                                     // the host start table is read by the copy above
  P.n_split = n_short / 16 * 16;
  dfree(g, cnt);
  dfree(g, cur);
}

// on_side: enqueue the kernels on the side stream after the buffers are
// allocated in main-stream order; group_by_shingle waits on ch.done (the
// chunk's keys and counters stay owned by the chunk until then).
void compute_chunk(sg_graph *g, PassOut &P, KeyChunk &ch, int st_hash, bool on_side = false) {
  if (!on_side) st_begin(g, st_hash);   // side chunks: timed on the side stream below
  dalloc(g, ch.keys, (size_t)ch.nt * (size_t)P.key_stride * 8);
  // top key bytes for the coarse histogram (1 B instead of 8 B per pair):
  // single rank, stable grouping, rows in generator order
  const bool want_kbin = P.kbin;
  if (want_kbin) dalloc(g, ch.kbin, (size_t)ch.nt * (size_t)P.key_stride);
  DBuf &ctr = ch.ctr;
  dalloc(g, ctr, 16);
  CK(cudaMemsetAsync(ctr.p, 0, 16, g->stream));
  cudaStream_t st = g->stream;
  if (on_side) {
    if (!ch.done) CK(cudaEventCreateWithFlags(&ch.done, cudaEventDisableTiming));
    CK(cudaEventRecord(ch.done, g->stream));          // buffers ready (main-stream order)
    CK(cudaStreamWaitEvent(g->side, ch.done, 0));
    st = g->side;
    st_begin(g, st_hash, st);
  }
  MinhashArgs a;
  const bool perm = P.perm.p != nullptr;
  a.rstart = ptr<int64_t>(perm ? P.rstart_p : P.rstart);
  a.rlen = ptr<int32_t>(perm ? P.rlen_p : P.rlen);
  a.entries = P.entries;
  a.nrows = P.nrows;
  a.A = ptr<uint32_t>(P.A);
  a.B = ptr<uint32_t>(P.B);
  a.t0 = ch.t0;
  a.nt = ch.nt;
  a.s = P.s;
  a.seed = P.seed;
  a.keys = ptr<uint64_t>(ch.keys);
  a.kbin = want_kbin ? ptr<uint8_t>(ch.kbin) : nullptr;
  a.key_stride = P.key_stride;
  a.counter = ptr<unsigned long long>(ctr);
  a.hub_counter = a.counter + 1;
  a.tile_rows = st_hash == kStHash2 ? 16 : 8;   // pass II rows are short
  if (perm && P.n_split > 0) {
    // rows of <= 8 entries one per lane, then the rest with the tile kernels
    MinhashArgs s = a;
    s.nrows = P.n_split;
    CK(minhash_short_rows(s, g->num_sms, st));
    a.rstart += P.n_split;
    a.rlen += P.n_split;
    a.keys += P.n_split;                       // n_split % 16 == 0: tile stores stay aligned
    a.nrows -= P.n_split;
  }
  CK(minhash(a, g->num_sms, st));
  if (on_side) {
    st_end(g, st_hash, st);
    CK(cudaEventRecord(ch.done, g->side));
  } else {
    dfree(g, ctr);
    st_end(g, st_hash);
  }
  ch.computed = true;
}

// ---------------------------------------------------------------- grouping
struct GroupScratch {
  DBuf p_trial, p_in0, p_len, p_row0, p_chunk0, seg, trial_chunk0;
  DBuf chunk_i0, chunk_in0, chunk_len, chunk_trial;
  DBuf counts, bstart1, bsize1, bstart, bsize, akeys, avals, bkeys, bvals, big_list, big_count;
  DBuf seg_pos, seg_len, fbin;
};

void free_scratch(sg_graph *g, GroupScratch &S) {
  for (DBuf *b : {&S.p_trial, &S.p_in0, &S.p_len, &S.p_row0, &S.p_chunk0, &S.seg, &S.trial_chunk0,
                  &S.chunk_i0, &S.chunk_in0, &S.chunk_len, &S.chunk_trial,
                  &S.counts, &S.bstart1, &S.bsize1, &S.bstart, &S.bsize, &S.akeys, &S.avals,
                  &S.bkeys, &S.bvals, &S.big_list, &S.big_count, &S.seg_pos, &S.seg_len, &S.fbin})
    dfree(g, *b);
}

bool use_group_v1();

// Scratch bytes per pair of a trial segment of `maxseg` pairs (planning).
double scratch_per_pair(int64_t maxseg) {
  if (!use_group_v1()) return 13.9;          // v3: one partitioned copy (8 B key + 4 B value) + segment list
  int32_t b, b1;
  group_bits(maxseg, &b, &b1);
  return b == b1 ? 12.5 : (b == 16 && b1 == 8 && getenv("SG_FBIN") ? 25.5 : 24.5);   // + fine bytes
}

// A contiguous run of pre-group pairs of one (local) trial: keys / explicit
// values at [in0, in0 + len), generator rows row0.. (implicit values).
struct Piece {
  int32_t trial;
  int64_t in0, len, row0;
};

void upload(sg_graph *g, DBuf &b, const void *h, size_t bytes) {
  if (b.bytes < std::max<size_t>(bytes, 16)) dalloc(g, b, bytes);
  if (bytes) CK(cudaMemcpyAsync(b.p, h, bytes, cudaMemcpyHostToDevice, g->stream));
}

void need(sg_graph *g, DBuf &b, size_t bytes) {
  if (b.bytes < std::max<size_t>(bytes, 16)) dalloc(g, b, bytes);
}

// Piece table of a partition over `nt` trials (pieces ordered by trial, then
// input order; chunks of <= group_chunk_pairs() pairs are found on the device
// by binary search over the pieces' first chunks).  Returns the chunk count.
int64_t build_pieces(sg_graph *g, const std::vector<Piece> &pieces, int32_t nt, GroupScratch &S,
                     GroupPlan &plan, int64_t CH = 0) {
  if (CH <= 0) CH = group_chunk_pairs();
  plan.chunk = CH;
  std::vector<int32_t> tr, tc0((size_t)nt + 1, 0);
  std::vector<int64_t> in0, len, row0, c0;
  int64_t nch = 0;
  size_t pi = 0;
  for (int j = 0; j < nt; ++j) {
    tc0[(size_t)j] = (int32_t)nch;
    for (; pi < pieces.size() && pieces[pi].trial == j; ++pi) {
      const Piece &p = pieces[pi];
      if (p.len <= 0) continue;
      tr.push_back(j);
      in0.push_back(p.in0);
      len.push_back(p.len);
      row0.push_back(p.row0);
      c0.push_back(nch);
      nch += (p.len + CH - 1) / CH;
    }
  }
  tc0[(size_t)nt] = (int32_t)nch;
  c0.push_back(nch);
  upload(g, S.p_trial, tr.data(), tr.size() * 4);
  upload(g, S.p_in0, in0.data(), in0.size() * 8);
  upload(g, S.p_len, len.data(), len.size() * 8);
  upload(g, S.p_row0, row0.data(), row0.size() * 8);
  upload(g, S.p_chunk0, c0.data(), c0.size() * 8);
  upload(g, S.trial_chunk0, tc0.data(), tc0.size() * 4);
  need(g, S.chunk_i0, (size_t)nch * 8);
  need(g, S.chunk_in0, (size_t)nch * 8);
  need(g, S.chunk_len, (size_t)nch * 4);
  need(g, S.chunk_trial, (size_t)nch * 4);
  plan.chunk_i0 = ptr<int64_t>(S.chunk_i0);
  plan.chunk_in0 = ptr<int64_t>(S.chunk_in0);
  plan.chunk_len = ptr<int32_t>(S.chunk_len);
  plan.chunk_trial = ptr<int32_t>(S.chunk_trial);
  plan.trial_chunk0 = ptr<int32_t>(S.trial_chunk0);
  plan.nchunks = nch;
  CK(group_chunk_tables(plan, ptr<int32_t>(S.p_trial), ptr<int64_t>(S.p_in0), ptr<int64_t>(S.p_len),
                        ptr<int64_t>(S.p_row0), ptr<int64_t>(S.p_chunk0), (int32_t)tr.size(),
                        g->stream));
  return nch;
}

// Group `nt` trials whose pairs are given as pieces into out.members /
// out.head (and okeys) at the global positions seg_all[t0 + j].
void group_pieces(sg_graph *g, const uint64_t *keys, const std::vector<Piece> &pieces, int32_t t0,
                  int32_t nt, const std::vector<int64_t> &seg_all, const uint32_t *vals,
                  const uint32_t *rowid, uint32_t val_base, Groups &out, uint64_t *okeys,
                  GroupScratch &S, DBuf *free_after_scatter, int st_hist, int st_scatter,
                  int st_local, const uint8_t *kbin = nullptr) {
  int64_t maxseg = 0, npairs = 0;
  for (int j = 0; j < nt; ++j) {
    const int64_t L = seg_all[(size_t)t0 + j + 1] - seg_all[(size_t)t0 + j];
    maxseg = std::max(maxseg, L);
    npairs += L;
  }
  if (maxseg >= (int64_t)0xFFFFFFFFll) fail(g, SG_EOVERFLOW, "a trial segment exceeds 2^32 pairs");
  // final buckets of ~1-2K pairs (the shared-memory sort holds 4K); the
  // coarse scatter fans out to <= 1024 buckets, a second level splits them
  // further for very long trial segments
  int32_t bits = 0, bits1 = 0;
  group_bits(maxseg, &bits, &bits1);
  const bool two = bits != bits1;
  const int64_t nbins = (int64_t)1 << bits;
  const int64_t nb1 = (int64_t)1 << bits1;
  GroupArgs a;
  const int64_t nch = build_pieces(g, pieces, nt, S, a.plan);
  std::vector<int64_t> seg((size_t)nt + 1);
  for (int j = 0; j <= nt; ++j) seg[(size_t)j] = seg_all[(size_t)t0 + j];
  upload(g, S.seg, seg.data(), seg.size() * 8);
  auto need = [&](DBuf &b, size_t bytes) { ::need(g, b, bytes); };
  need(S.counts, (size_t)(nch * nb1) * 4);
  need(S.bstart1, (size_t)(nt * nb1) * 4);
  need(S.bsize1, (size_t)(nt * nb1) * 4);
  need(S.akeys, (size_t)npairs * 8);
  need(S.avals, (size_t)npairs * 4);
  // fine digits as bytes for the fine split's histogram (16-bit plans)
  // (opt-in SG_FBIN=1: measured on gos2m fine 67.3 -> 62.9 ms but the
  // coarse scatter's byte stores 76.7 -> 82.5 ms)
  const bool fb = two && bits == 16 && bits1 == 8 && getenv("SG_FBIN");
  if (two) {
    need(S.bstart, (size_t)(nt * nbins) * 4);
    need(S.bsize, (size_t)(nt * nbins) * 4);
    need(S.bkeys, (size_t)npairs * 8);
    need(S.bvals, (size_t)npairs * 4);
    if (fb) need(S.fbin, (size_t)npairs);
  }
  need(S.big_list, (size_t)(nt * nbins) * 8);             // big + mid lists
  need(S.big_count, 8);                                    // big + mid counts
  CK(cudaMemsetAsync(S.big_count.p, 0, 8, g->stream));
  a.plan.c = nt;
  a.plan.bits = bits;
  a.plan.bits1 = bits1;
  a.plan.nbins = nbins;
  a.plan.nb1 = nb1;
  a.plan.npairs = npairs;
  a.plan.seg = ptr<int64_t>(S.seg);
  a.keys = keys;
  a.kbin = kbin;
  a.vals = vals;
  a.rowid = rowid;
  a.val_base = val_base;
  a.counts = ptr<uint32_t>(S.counts);
  a.bstart1 = ptr<uint32_t>(S.bstart1);
  a.bsize1 = ptr<uint32_t>(S.bsize1);
  a.akeys = ptr<uint64_t>(S.akeys);
  a.avals = ptr<uint32_t>(S.avals);
  a.bstart = two ? ptr<uint32_t>(S.bstart) : a.bstart1;
  a.bsize = two ? ptr<uint32_t>(S.bsize) : a.bsize1;
  a.bkeys = two ? ptr<uint64_t>(S.bkeys) : a.akeys;
  a.bvals = two ? ptr<uint32_t>(S.bvals) : a.avals;
  a.fbin = fb ? ptr<uint8_t>(S.fbin) : nullptr;
  a.big_list = ptr<uint32_t>(S.big_list);
  a.big_count = ptr<uint32_t>(S.big_count);
  a.mid_list = a.big_list + nt * nbins;
  a.mid_count = a.big_count + 1;
  a.members = ptr<uint32_t>(out.members);
  a.head = ptr<uint32_t>(out.head);
  a.okeys = okeys;
  st_begin(g, st_hist);
  CK(group_hist(a, g->stream));
  CK(group_offsets(a, g->stream));
  st_end(g, st_hist);
  st_begin(g, st_scatter);
  CK(group_scatter(a, g->num_sms, g->stream));
  if (free_after_scatter) dfree(g, *free_after_scatter);   // keys consumed
  st_end(g, st_scatter);
  if (two) {
    st_begin(g, st_scatter == kStScatter1 ? kStFine1 : kStFine2);
    CK(group_scatter2(a, g->stream));
    st_end(g, st_scatter == kStScatter1 ? kStFine1 : kStFine2);
  }
  st_begin(g, st_local);
  CK(group_local(a, g->num_sms, g->stream));
  st_end(g, st_local);
}

// Grouping design: the stable two-level partition + warp /
// CTA local sorts (group_pieces, the default: measured fastest) or, with
// SG_GROUP=v3, the order-independent design of kernels_sort.cu (coarse
// atomic scatter + per-bucket counting sort + segmented member sort; parity-
// green, measured slower; kept as the A/B alternative it was measured as).
bool use_group_v1() {
  const char *e = getenv("SG_GROUP");
  return !(e && strcmp(e, "v3") == 0);
}

void group_pieces_b(sg_graph *g, const uint64_t *keys, const std::vector<Piece> &pieces, int32_t t0,
                    int32_t nt, const std::vector<int64_t> &seg_all, const uint32_t *vals,
                    const uint32_t *rowid, uint32_t val_base, Groups &out, uint64_t *okeys,
                    GroupScratch &S, DBuf *free_after_scatter, int st_hist, int st_scatter,
                    int st_local) {
  int64_t maxseg = 0, npairs = 0;
  for (int j = 0; j < nt; ++j) {
    const int64_t L = seg_all[(size_t)t0 + j + 1] - seg_all[(size_t)t0 + j];
    maxseg = std::max(maxseg, L);
    npairs += L;
  }
  if (maxseg >= (int64_t)0xFFFFFFFFll) fail(g, SG_EOVERFLOW, "a trial segment exceeds 2^32 pairs");
  int32_t bits1 = 0, fine = 0;
  group_c_bits(maxseg, &bits1, &fine);
  const int64_t nb = (int64_t)1 << bits1;
  GroupArgs a;
  build_pieces(g, pieces, nt, S, a.plan, group_c_chunk_pairs());
  std::vector<int64_t> seg((size_t)nt + 1);
  for (int j = 0; j <= nt; ++j) seg[(size_t)j] = seg_all[(size_t)t0 + j];
  upload(g, S.seg, seg.data(), seg.size() * 8);
  need(g, S.bstart1, (size_t)(nt * nb) * 4);
  need(g, S.bsize1, (size_t)(nt * nb) * 4);
  need(g, S.counts, (size_t)(nt * nb) * 4);          // the scatter's reservation cursors
  need(g, S.akeys, (size_t)npairs * 8);
  need(g, S.avals, (size_t)npairs * 4);
  const int64_t scr = group_c_scratch_pairs(g->num_sms);
  need(g, S.bkeys, (size_t)scr * 8);
  need(g, S.bvals, (size_t)scr * 4);
  need(g, S.big_list, (size_t)(nt * nb) * 4);
  need(g, S.big_count, 16);
  CK(cudaMemsetAsync(S.big_count.p, 0, 16, g->stream));
  const int64_t nseg = npairs / 9 + 1;                 // one-key fine buckets of >= 9 members
  need(g, S.seg_pos, (size_t)nseg * 8);
  need(g, S.seg_len, (size_t)nseg * 4);
  a.plan.c = nt;
  a.plan.bits = bits1;
  a.plan.bits1 = bits1;
  a.plan.nbins = nb;
  a.plan.nb1 = nb;
  a.plan.fine_bits = fine;
  a.plan.npairs = npairs;
  a.plan.seg = ptr<int64_t>(S.seg);
  if (const char *lc = getenv("SG_LOCAL_CAP")) a.plan.local_cap = atoi(lc);   // test hook
  a.keys = keys;
  a.vals = vals;
  a.rowid = rowid;
  a.val_base = val_base;
  a.bstart1 = a.bstart = ptr<uint32_t>(S.bstart1);
  a.bsize1 = a.bsize = ptr<uint32_t>(S.bsize1);
  a.gcur = ptr<uint32_t>(S.counts);
  a.akeys = ptr<uint64_t>(S.akeys);
  a.avals = ptr<uint32_t>(S.avals);
  a.bkeys = ptr<uint64_t>(S.bkeys);
  a.bvals = ptr<uint32_t>(S.bvals);
  a.big_list = ptr<uint32_t>(S.big_list);
  a.big_count = ptr<uint32_t>(S.big_count);
  a.seg_count = reinterpret_cast<unsigned long long *>(ptr<uint32_t>(S.big_count) + 2);
  a.seg_pos = ptr<int64_t>(S.seg_pos);
  a.seg_len = ptr<uint32_t>(S.seg_len);
  a.members = ptr<uint32_t>(out.members);
  a.head = ptr<uint32_t>(out.head);
  a.okeys = okeys;
  st_begin(g, st_hist);
  CK(group_c_hist(a, g->num_sms, g->stream));
  st_end(g, st_hist);
  st_begin(g, st_scatter);
  CK(group_c_scatter(a, g->num_sms, g->stream));
  if (free_after_scatter) dfree(g, *free_after_scatter);   // keys consumed
  st_end(g, st_scatter);
  st_begin(g, st_local);
  CK(group_c_bucket(a, g->num_sms, g->stream));
  CK(group_c_segsort(a, g->num_sms, g->stream));
  st_end(g, st_local);
}

void group_any(sg_graph *g, const uint64_t *keys, const std::vector<Piece> &pieces, int32_t t0,
               int32_t nt, const std::vector<int64_t> &seg_all, const uint32_t *vals,
               const uint32_t *rowid, uint32_t val_base, Groups &out, uint64_t *okeys,
               GroupScratch &S, DBuf *free_after_scatter, int st_hist, int st_scatter, int st_local,
               const uint8_t *kbin = nullptr) {
  if (use_group_v1())
    group_pieces(g, keys, pieces, t0, nt, seg_all, vals, rowid, val_base, out, okeys, S,
                 free_after_scatter, st_hist, st_scatter, st_local, kbin);
  else
    group_pieces_b(g, keys, pieces, t0, nt, seg_all, vals, rowid, val_base, out, okeys, S,
                   free_after_scatter, st_hist, st_scatter, st_local);
}

int64_t device_sum_popc(sg_graph *g, const DBuf &words, int64_t nwords) {
  if (nwords == 0) return 0;
  DBuf d;
  dalloc(g, d, 8);
  CK(popcount_words(ptr<uint32_t>(words), nwords, ptr<unsigned long long>(d), g->stream));
  unsigned long long h = 0;
  CK(cudaMemcpyAsync(&h, d.p, 8, cudaMemcpyDeviceToHost, g->stream));
  sync(g);
  dfree(g, d);
  return (int64_t)h;
}

template <typename T>
std::vector<T> d2h(sg_graph *g, const DBuf &b, size_t count) {
  std::vector<T> v(count);
  if (count) {
    CK(cudaMemcpyAsync(v.data(), b.p, count * sizeof(T), cudaMemcpyDeviceToHost, g->stream));
    sync(g);
  }
  return v;
}

// Recompute shingle ids of (row, trial) requests of pass `level` on device.
std::vector<uint64_t> recompute_ids(sg_graph *g, int level, const std::vector<int64_t> &rows,
                                    const std::vector<int32_t> &trials) {
  PassOut &P = g->pass[level];
  const size_t nq = rows.size();
  std::vector<uint64_t> out(nq);
  if (!nq) return out;
  DBuf dr, dt, di;
  dalloc(g, dr, nq * 8);
  dalloc(g, dt, nq * 4);
  dalloc(g, di, nq * 8);
  CK(cudaMemcpyAsync(dr.p, rows.data(), nq * 8, cudaMemcpyHostToDevice, g->stream));
  CK(cudaMemcpyAsync(dt.p, trials.data(), nq * 4, cudaMemcpyHostToDevice, g->stream));
  CK(shingle_ids(ptr<int64_t>(P.rstart), ptr<int32_t>(P.rlen), P.entries, ptr<uint32_t>(P.A),
                 ptr<uint32_t>(P.B), P.s, P.seed, ptr<int64_t>(dr), ptr<int32_t>(dt),
                 (int64_t)nq, ptr<uint64_t>(di), g->stream));
  CK(cudaMemcpyAsync(out.data(), di.p, nq * 8, cudaMemcpyDeviceToHost, g->stream));
  sync(g);
  dfree(g, dr);
  dfree(g, dt);
  dfree(g, di);
  return out;
}

// ---------------------------------------------------------------- multi-rank
[[noreturn]] void require_single(sg_graph *g, const std::string &what) {
  fail(g, SG_EINVAL, what + " needs world == 1 (gather the per-rank groups with the getters)");
}

// Pass-II dense index k, identical for every world size: S1' nodes are ordered
// by (pass-I trial j, key) and key ranges are ordered by rank, so the local
// S1' rows of trial j (rows [first_j, first_{j+1})) get
// k = K_j + sum_{r' < rank} S[j][r'] + (i - first_j).
void assign_s1p_index(sg_graph *g, PassOut &P) {
  Groups &G1 = g->grp[0];
  const int c1 = G1.c, R = g->world, me = g->rank;
  DBuf dseg, dcnt, dfirst, doff;
  upload(g, dseg, G1.seg.data(), G1.seg.size() * 8);
  dalloc(g, dcnt, (size_t)c1 * 8);
  CK(cudaMemsetAsync(dcnt.p, 0, (size_t)c1 * 8, g->stream));
  CK(rows_per_trial(ptr<int64_t>(P.rstart), P.nrows, ptr<int64_t>(dseg), c1,
                    ptr<unsigned long long>(dcnt), g->stream));
  std::vector<int64_t> cnt = d2h<int64_t>(g, dcnt, (size_t)c1);
  std::vector<int64_t> all((size_t)c1 * R);
  x_allgather_i64(g, cnt.data(), c1, all.data());
  std::vector<int64_t> first((size_t)c1 + 1), off((size_t)c1);
  int64_t K = 0;
  sg_s1p_offsets(R, me, c1, all.data(), first.data(), off.data(), &K);
  g->s1p_global = K;
  g->s1p_k0 = -1;                       // the local k values are not one range
  P.blocks = first;                     // rows grouped by pass-I trial
  upload(g, dfirst, first.data(), first.size() * 8);
  upload(g, doff, off.data(), off.size() * 8);
  dalloc(g, P.rowid, (size_t)P.nrows * 4);
  CK(assign_rowid(ptr<uint32_t>(P.rowid), P.nrows, ptr<int64_t>(dfirst), ptr<int64_t>(doff), c1,
                  g->stream));
  for (DBuf *b : {&dseg, &dcnt, &dfirst, &doff}) dfree(g, *b);
}

// Owner partition of one key chunk: pairs of (trial tl, row block b) go to
// rank owner(key) = floor(key * R / 2^64) (contiguous key ranges, so the
// canonical key order is rank-major).  Virtual trial vt = tl * nblk + b.
// Phase `starts == nullptr`: counts only (mine[vt * R + d]).  Otherwise the
// pairs are written dest-major (then vt, then row order) into skeys / svals.
// Fused exchange (SG_DIST_PEER): peer_k / peer_v are device arrays of the
// owners' receive buffers and `starts` are positions in them; the pairs are
// stored there directly (skeys / svals unused).
void owner_partition(sg_graph *g, PassOut &P, KeyChunk &ch, GroupScratch &S,
                     std::vector<int64_t> *mine, const std::vector<int64_t> *starts,
                     uint64_t *skeys, uint32_t *svals, uint64_t *const *peer_k = nullptr,
                     uint32_t *const *peer_v = nullptr) {
  const int R = g->world;
  const std::vector<int64_t> &Bk = P.blocks;
  const int nblk = (int)Bk.size() - 1;
  const int nvt = ch.nt * nblk;
  std::vector<Piece> pieces;
  for (int tl = 0; tl < ch.nt; ++tl)
    for (int b = 0; b < nblk; ++b)
      if (Bk[(size_t)b + 1] > Bk[(size_t)b])
        pieces.push_back(Piece{tl * nblk + b, (int64_t)tl * P.key_stride + Bk[(size_t)b],
                               Bk[(size_t)b + 1] - Bk[(size_t)b], Bk[(size_t)b]});
  GroupArgs a;
  const int64_t nch = build_pieces(g, pieces, nvt, S, a.plan);
  need(g, S.counts, (size_t)(nch * R) * 4);
  need(g, S.bsize1, (size_t)nvt * R * 4);
  need(g, S.bstart1, (size_t)nvt * R * 4);
  a.plan.c = nvt;
  a.plan.nb1 = R;
  a.plan.nbins = R;
  a.keys = ptr<uint64_t>(ch.keys);
  a.vals = nullptr;
  a.rowid = ptr<uint32_t>(P.rowid);
  a.val_base = 0;
  a.counts = ptr<uint32_t>(S.counts);
  a.bsize1 = ptr<uint32_t>(S.bsize1);
  a.bstart1 = ptr<uint32_t>(S.bstart1);
  CK(group_hist(a, g->stream));
  CK(group_colscan(a, g->stream));
  if (!starts) {
    std::vector<uint32_t> bs = d2h<uint32_t>(g, S.bsize1, (size_t)nvt * R);
    mine->assign(bs.begin(), bs.end());
    return;
  }
  for (int64_t v : *starts)
    if (v > (int64_t)UINT32_MAX) fail(g, SG_EOVERFLOW, "a send buffer of one trial chunk exceeds 2^32 pairs");
  std::vector<uint32_t> st32(starts->begin(), starts->end());
  upload(g, S.bstart1, st32.data(), st32.size() * 4);
  std::vector<int64_t> zeros((size_t)nvt + 1, 0);
  upload(g, S.seg, zeros.data(), zeros.size() * 8);
  a.plan.seg = ptr<int64_t>(S.seg);
  a.akeys = skeys;
  a.avals = svals;
  a.peer_keys = peer_k;
  a.peer_vals = peer_v;
  CK(group_scatter(a, g->num_sms, g->stream));
}

// Receive buffers of the fused exchange: cudaMalloc'd (IPC-exportable), one
// pair per level, mapped by every rank; released on every exit path.
struct PeerRecv {
  void *k = nullptr, *v = nullptr;
  std::vector<void *> opened;
  DBuf dk, dv;                 // device arrays of the R peer pointers
  ~PeerRecv() {
    for (void *p : opened) cudaIpcCloseMemHandle(p);
    if (k) cudaFree(k);
    if (v) cudaFree(v);
  }
};

// Exchange + grouping of one level on a multi-rank handle.
void group_multi(sg_graph *g, int level) {
  PassOut &P = g->pass[level];
  Groups &out = g->grp[level];
  const int c = P.c, R = g->world, me = g->rank;
  const int nblk = (int)P.blocks.size() - 1;
  const int st_x = level == 0 ? kStX1 : kStX2;
  GroupScratch S;
  // phase 1: owner counts of every chunk, exchanged (all ranks: all chunks)
  std::vector<std::vector<int64_t>> mine(P.chunks.size()), all(P.chunks.size());
  for (size_t k = 0; k < P.chunks.size(); ++k) {
    KeyChunk &ch = P.chunks[k];
    if (!ch.computed) compute_chunk(g, P, ch, level == 0 ? kStHash1 : kStHash2);
    st_begin(g, st_x);
    owner_partition(g, P, ch, S, &mine[k], nullptr, nullptr, nullptr);
    const int64_t n = (int64_t)ch.nt * nblk * R;
    all[k].resize((size_t)n * R);
    x_allgather_i64(g, mine[k].data(), n, all[k].data());
    st_end(g, st_x);
  }
  // local trial segments of the received pairs
  free_groups(g, out);
  out.c = c;
  out.seg.assign((size_t)c + 1, 0);
  for (size_t k = 0; k < P.chunks.size(); ++k) {
    const KeyChunk &ch = P.chunks[k];
    const int64_t n = (int64_t)ch.nt * nblk * R;
    for (int tl = 0; tl < ch.nt; ++tl) {
      int64_t tot = 0;
      for (int s = 0; s < R; ++s)
        for (int b = 0; b < nblk; ++b) tot += all[k][(size_t)(s * n + ((int64_t)tl * nblk + b) * R + me)];
      out.seg[(size_t)ch.t0 + tl + 1] = tot;
    }
  }
  for (int j = 0; j < c; ++j) out.seg[(size_t)j + 1] += out.seg[(size_t)j];
  out.npairs = out.seg[(size_t)c];
  dalloc(g, out.members, (size_t)out.npairs * 4);
  dalloc(g, out.okeys, (size_t)out.npairs * 8);
  dalloc(g, out.head, (size_t)((out.npairs + 31) / 32) * 4);
  CK(cudaMemsetAsync(out.head.p, 0, out.head.bytes, g->stream));
  // fused exchange: one receive buffer per rank, sized for its largest chunk
  PeerRecv pr;
  if (g->peer_xch) {
    int64_t rcap = 1;
    for (size_t k = 0; k < P.chunks.size(); ++k) {
      const int64_t n = (int64_t)P.chunks[k].nt * nblk * R;
      int64_t t = 0;
      for (int s = 0; s < R; ++s)
        for (int64_t vt = 0; vt < (int64_t)P.chunks[k].nt * nblk; ++vt)
          t += all[k][(size_t)(s * n + vt * R + me)];
      rcap = std::max(rcap, t);
    }
    CK(cudaMalloc(&pr.k, (size_t)rcap * 8));
    CK(cudaMalloc(&pr.v, (size_t)rcap * 4));
    void *mine2[2] = {pr.k, pr.v};
    std::vector<void *> peers;
    x_share_buffers(g, mine2, 2, peers, pr.opened);
    std::vector<void *> pk((size_t)R), pv((size_t)R);
    for (int r = 0; r < R; ++r) {
      pk[(size_t)r] = peers[(size_t)r * 2];
      pv[(size_t)r] = peers[(size_t)r * 2 + 1];
    }
    upload(g, pr.dk, pk.data(), (size_t)R * sizeof(void *));
    upload(g, pr.dv, pv.data(), (size_t)R * sizeof(void *));
  }
  // phase 2: per chunk, partition to send buffers, all-to-all, group
  for (size_t k = 0; k < P.chunks.size(); ++k) {
    KeyChunk &ch = P.chunks[k];
    const int nvt = ch.nt * nblk;
    const int64_t n = (int64_t)nvt * R;
    const std::vector<int64_t> &my = mine[k];
    std::vector<int64_t> soff((size_t)R + 1, 0), starts((size_t)nvt * R);
    for (int d = 0; d < R; ++d) {
      int64_t run = soff[(size_t)d];
      for (int vt = 0; vt < nvt; ++vt) {
        starts[(size_t)vt * R + d] = run;
        run += my[(size_t)vt * R + d];
      }
      soff[(size_t)d + 1] = run;
    }
    std::vector<int64_t> roff((size_t)R + 1, 0);
    for (int s = 0; s < R; ++s) {
      int64_t t = 0;
      for (int vt = 0; vt < nvt; ++vt) t += all[k][(size_t)(s * n + (int64_t)vt * R + me)];
      roff[(size_t)s + 1] = roff[(size_t)s] + t;
    }
    DBuf skeys, svals, rkeys, rvals;
    uint64_t *rk = nullptr;
    uint32_t *rv = nullptr;
    if (g->peer_xch) {
      // positions in the owners' receive buffers (their layout: source-major,
      // then virtual trial, then row order — the send / recv layout)
      std::vector<int64_t> pst((size_t)nvt * R);
      for (int d = 0; d < R; ++d) {
        int64_t run = 0;
        for (int s = 0; s < me; ++s)
          for (int vt = 0; vt < nvt; ++vt) run += all[k][(size_t)(s * n + (int64_t)vt * R + d)];
        for (int vt = 0; vt < nvt; ++vt) {
          pst[(size_t)vt * R + d] = run;
          run += all[k][(size_t)(me * n + (int64_t)vt * R + d)];
        }
      }
      st_begin(g, st_x);
      x_barrier(g);                    // every owner has grouped its previous chunk
      owner_partition(g, P, ch, S, nullptr, &pst, nullptr, nullptr,
                      reinterpret_cast<uint64_t *const *>(pr.dk.p),
                      reinterpret_cast<uint32_t *const *>(pr.dv.p));
      dfree(g, ch.keys);
      ch.computed = false;
      sync(g);
      x_barrier(g);                    // every pair of this chunk is delivered
      st_end(g, st_x);
      rk = static_cast<uint64_t *>(pr.k);
      rv = static_cast<uint32_t *>(pr.v);
    } else {
      dalloc(g, skeys, (size_t)soff[(size_t)R] * 8);
      dalloc(g, svals, (size_t)soff[(size_t)R] * 4);
      dalloc(g, rkeys, (size_t)roff[(size_t)R] * 8);
      dalloc(g, rvals, (size_t)roff[(size_t)R] * 4);
      st_begin(g, st_x);
      owner_partition(g, P, ch, S, nullptr, &starts, ptr<uint64_t>(skeys), ptr<uint32_t>(svals));
      dfree(g, ch.keys);
      ch.computed = false;
      x_alltoallv2(g, skeys.p, rkeys.p, 8, svals.p, rvals.p, 4, soff.data(), roff.data());
      st_end(g, st_x);
      dfree(g, skeys);
      dfree(g, svals);
      rk = ptr<uint64_t>(rkeys);
      rv = ptr<uint32_t>(rvals);
    }
    // received pieces in canonical generator order: trial, row block, source
    std::vector<Piece> pieces;
    for (int tl = 0; tl < ch.nt; ++tl)
      for (int b = 0; b < nblk; ++b)
        for (int s = 0; s < R; ++s) {
          const int vt = tl * nblk + b;
          int64_t o = roff[(size_t)s];
          for (int v2 = 0; v2 < vt; ++v2) o += all[k][(size_t)(s * n + (int64_t)v2 * R + me)];
          const int64_t len = all[k][(size_t)(s * n + (int64_t)vt * R + me)];
          if (len > 0) pieces.push_back(Piece{tl, o, len, 0});
        }
    group_any(g, rk, pieces, ch.t0, ch.nt, out.seg, rv,
                 nullptr, 0, out, ptr<uint64_t>(out.okeys), S, nullptr,
                 level == 0 ? kStHist1 : kStHist2, level == 0 ? kStScatter1 : kStScatter2,
                 level == 0 ? kStLocal1 : kStLocal2);
    if (rkeys.p) dfree(g, rkeys);
    if (rvals.p) dfree(g, rvals);
  }
  if (g->peer_xch) {
    sync(g);                           // this rank's reads of its receive buffer are done
    x_release_buffers(g, pr.opened);   // barrier: no peer writes any more
    dfree(g, pr.dk);
    dfree(g, pr.dv);
  }
  free_scratch(g, S);
  g->pairs_global[level] = exchange_sum(g, out.npairs);
}

// Host view of trials [t0, t1) of a grouped level: per-trial group ranges,
// group offsets (relative to the first pair of trial t0), ids.
struct HostGroups {
  std::vector<int64_t> trial_goffs, offs;
  std::vector<uint64_t> ids;
  std::vector<uint32_t> members;
};

template <typename T>
std::vector<T> d2h_range(sg_graph *g, const DBuf &b, size_t first, size_t count) {
  std::vector<T> v(count);
  if (count) {
    CK(cudaMemcpyAsync(v.data(), reinterpret_cast<const T *>(b.p) + first, count * sizeof(T),
                       cudaMemcpyDeviceToHost, g->stream));
    sync(g);
  }
  return v;
}

void host_groups(sg_graph *g, int level, HostGroups &H, bool want_ids, int t0 = 0, int t1 = -1) {
  Groups &q = g->grp[level];
  PassOut &p = g->pass[level];
  if (t1 < 0) t1 = q.c;
  const int nt = t1 - t0;
  const int64_t p0 = q.seg[(size_t)t0], p1 = q.seg[(size_t)t1], np = p1 - p0;
  H.members = d2h_range<uint32_t>(g, q.members, (size_t)p0, (size_t)np);
  const int64_t w0 = p0 >> 5, w1 = (p1 + 31) >> 5;
  std::vector<uint32_t> head = d2h_range<uint32_t>(g, q.head, (size_t)w0, (size_t)(w1 - w0));
  H.trial_goffs.assign((size_t)nt + 1, 0);
  H.offs.clear();
  int j = 0;
  for (int64_t i = p0; i < p1; ++i) {
    while (j < nt && q.seg[(size_t)t0 + j + 1] <= i) {
      ++j;
      H.trial_goffs[(size_t)j] = (int64_t)H.offs.size();
    }
    if ((head[(size_t)((i >> 5) - w0)] >> (i & 31)) & 1u) H.offs.push_back(i - p0);
  }
  while (j < nt) {
    ++j;
    H.trial_goffs[(size_t)j] = (int64_t)H.offs.size();
  }
  const int64_t G = (int64_t)H.offs.size();
  H.offs.push_back(np);
  if (!want_ids) return;
  if (q.okeys.p) {
    // multi-rank: the grouping kept the sorted keys; id = fmix^-1(key)
    H.ids.resize((size_t)G);
    std::vector<uint64_t> ok = d2h_range<uint64_t>(g, q.okeys, (size_t)p0, (size_t)np);
    for (int64_t x = 0; x < G; ++x) H.ids[(size_t)x] = fmix_inv(ok[(size_t)H.offs[(size_t)x]]);
    return;
  }
  // id of a group = the shingle of its first (smallest) generator in that trial
  std::vector<uint32_t> rid;
  if (level == 0) rid = d2h<uint32_t>(g, p.rowid, (size_t)p.nrows);
  std::vector<int64_t> rows((size_t)G);
  std::vector<int32_t> trials((size_t)G);
  for (int jj = 0; jj < nt; ++jj) {
    for (int64_t x = H.trial_goffs[(size_t)jj]; x < H.trial_goffs[(size_t)jj + 1]; ++x) {
      const uint32_t m = H.members[(size_t)H.offs[(size_t)x]];
      rows[(size_t)x] = level == 0 ? (int64_t)(std::lower_bound(rid.begin(), rid.end(), m) - rid.begin())
                                   : (int64_t)m - g->s1p_k0;
      trials[(size_t)x] = t0 + jj;
    }
  }
  H.ids = recompute_ids(g, level, rows, trials);
}

// Copy this rank's row range of a host (or device) CSR into HBM, rebase it
// and validate it on the device (create and load).
void unmap_col(sg_graph *g) {
  if (g->col_reg) cudaHostUnregister(g->col_reg);
  cudaGetLastError();
  g->col_reg = nullptr;
  g->col_dev = nullptr;
}

void ingest(sg_graph *g, int64_t n, int64_t nnz, const int64_t *row_ptr, const int64_t *rp_host,
            const int32_t *col, bool devptr, bool validate, bool host_csr = false) {
  g->n = n;
  g->nnz_global = nnz;
  // row range of this rank
  std::vector<int64_t> bounds((size_t)g->world + 1);
  if (n > 0) sg_partition_rows(n, rp_host, g->world, 8, bounds.data());
  else std::fill(bounds.begin(), bounds.end(), 0);
  g->row_lo = bounds[(size_t)g->rank];
  g->row_hi = bounds[(size_t)g->rank + 1];
  const int64_t rows = g->row_hi - g->row_lo;
  const int64_t e0 = n > 0 ? rp_host[g->row_lo] : 0;
  const int64_t e1 = n > 0 ? rp_host[g->row_hi] : 0;
  // the copy below reads col[e0, e1) of the caller's buffer: check the
  // slice on the host first (validation proper runs on the device)
  if (e0 < 0 || e1 < e0 || e1 > nnz) fail(g, SG_EINVAL, "invalid CSR: row_ptr is not monotone within [0, nnz]");
  g->nnz_local = e1 - e0;
  dalloc(g, g->row_ptr, (size_t)(rows + 1) * 8);
  unmap_col(g);
  const bool mapped = host_csr && !devptr;
  if (mapped) {
    // out-of-core entries: page-lock and map the caller's slice; the kernels
    // read it over the host link (N4)
    dfree(g, g->col);
    if (g->nnz_local) {
      void *h = const_cast<int32_t *>(col + e0);
      cudaError_t e = cudaHostRegister(h, (size_t)g->nnz_local * 4,
                                       cudaHostRegisterMapped | cudaHostRegisterReadOnly);
      if (e == cudaErrorHostMemoryAlreadyRegistered) cudaGetLastError();   // the caller pinned it
      else {
        CK(e);
        g->col_reg = h;
      }
      void *d = nullptr;
      CK(cudaHostGetDevicePointer(&d, h, 0));
      g->col_dev = reinterpret_cast<const uint32_t *>(d);
    } else {
      dalloc(g, g->col, 16);
      g->col_dev = ptr<uint32_t>(g->col);
    }
  } else {
    dalloc(g, g->col, (size_t)g->nnz_local * 4);
    g->col_dev = ptr<uint32_t>(g->col);
  }
  const cudaMemcpyKind kind = devptr ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice;
  if (n > 0) {
    CK(cudaMemcpyAsync(g->row_ptr.p, row_ptr + g->row_lo, (rows + 1) * 8, kind, g->stream));
    if (g->nnz_local && !mapped)
      CK(cudaMemcpyAsync(g->col.p, col + e0, g->nnz_local * 4, kind, g->stream));
    rebase_kernel<<<std::min<int64_t>((rows + 256) / 256, 4096), 256, 0, g->stream>>>(
        ptr<int64_t>(g->row_ptr), rows + 1, e0);
    CK(cudaGetLastError());
  } else {
    CK(cudaMemsetAsync(g->row_ptr.p, 0, 8, g->stream));
  }
  if (validate && rows > 0) {
    // the CSR is validated on the device after the copy (O(nnz), one pass)
    DBuf bad;
    dalloc(g, bad, 4);
    CK(cudaMemsetAsync(bad.p, 0, 4, g->stream));
    validate_kernel<<<std::min<int64_t>((rows + 7) / 8, (int64_t)g->num_sms * 16), 256, 0, g->stream>>>(
        ptr<int64_t>(g->row_ptr), reinterpret_cast<const int32_t *>(g->col_dev), rows,
        g->nnz_local, n, ptr<int>(bad));
    CK(cudaGetLastError());
    int hb = 0;
    CK(cudaMemcpyAsync(&hb, bad.p, 4, cudaMemcpyDeviceToHost, g->stream));
    sync(g);
    dfree(g, bad);
    if (hb) fail(g, SG_EINVAL, "invalid CSR: a row is not strictly increasing, or an id is outside [0, n)");
  }
}

}  // namespace

// =============================================================================
extern "C" {

const char *sg_version(void) { return "libshingle 0.2 (sm_100a)"; }

const char *sg_last_error(const sg_graph *g) { return g ? g->err.c_str() : t_err.c_str(); }

sg_status sg_partition_rows(int64_t n, const int64_t *row_ptr, int32_t world, int64_t kappa,
                            int64_t *bounds) {
  if (n < 0 || world < 1 || !row_ptr || !bounds) return SG_EINVAL;
  // balance sum(deg + kappa): bounds[r] = first row whose prefix weight
  // reaches r/world of the total
  const long double tot = (long double)row_ptr[n] + (long double)kappa * (long double)n;
  bounds[0] = 0;
  int64_t u = 0;
  for (int32_t r = 1; r < world; ++r) {
    const long double target = tot * r / world;
    while (u < n && (long double)row_ptr[u] + (long double)kappa * u < target) ++u;
    bounds[r] = u;
  }
  bounds[world] = n;
  return SG_OK;
}

sg_status sg_s1p_offsets(int32_t world, int32_t rank, int32_t c1, const int64_t *all,
                         int64_t *first, int64_t *off, int64_t *total) {
  if (world < 1 || rank < 0 || rank >= world || c1 < 0 || !all || !first || !off) return SG_EINVAL;
  int64_t K = 0, f = 0;
  for (int j = 0; j < c1; ++j) {
    int64_t before = 0, sum = 0;
    for (int r = 0; r < world; ++r) {
      const int64_t v = all[(int64_t)r * c1 + j];
      if (r < rank) before += v;
      sum += v;
    }
    first[j] = f;
    off[j] = K + before - f;
    f += all[(int64_t)rank * c1 + j];
    K += sum;
  }
  first[c1] = f;
  if (total) *total = K;
  return SG_OK;
}

sg_status shingle_graph_create(int64_t n, int64_t nnz, const int64_t *row_ptr, const int32_t *col,
                               uint32_t flags, const sg_dist *dist, sg_graph **out) {
  if (!out) {
    t_err = "out is NULL";
    return SG_EINVAL;
  }
  *out = nullptr;
  if (n < 0 || (uint64_t)n >= kP || nnz < 0 || (n > 0 && !row_ptr) || (nnz > 0 && !col)) {
    t_err = "invalid n / nnz / pointers (need 0 <= n < 2^31 - 1)";
    return SG_EINVAL;
  }
  if (dist && (dist->world < 1 || dist->rank < 0 || dist->rank >= dist->world)) {
    t_err = "invalid sg_dist rank/world";
    return SG_EINVAL;
  }
  const bool devptr = flags & SG_DEVICE_PTRS;
  const bool validate = !(flags & SG_NO_VALIDATE);
  std::vector<int64_t> hrp;
  const int64_t *rp_host = row_ptr;
  if (devptr && n > 0) {
    // the partition needs the row pointers on the host (n+1 words, untimed)
    hrp.resize((size_t)n + 1);
    if (cudaMemcpy(hrp.data(), row_ptr, (n + 1) * 8, cudaMemcpyDeviceToHost) != cudaSuccess) {
      cudaGetLastError();
      t_err = "cannot read device row_ptr";
      return SG_EINVAL;
    }
    rp_host = hrp.data();
  }
  if (n > 0 && (rp_host[0] != 0 || rp_host[n] != nnz)) {
    t_err = "invalid CSR: row_ptr[0] must be 0 and row_ptr[n] must equal nnz";
    return SG_EINVAL;
  }
  std::unique_ptr<sg_graph> G(new sg_graph());
  sg_graph *g = G.get();
  g->n = n;
  g->nnz_global = nnz;
  g->rank = dist ? dist->rank : 0;
  g->world = dist ? dist->world : 1;
  if (const char *mb = getenv("SG_MEM_BUDGET")) g->mem_budget = atoll(mb);
  sg_status st = SG_OK;
  try {
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) {
      cudaGetLastError();
      fail(g, SG_ECUDA, "no CUDA device available (libshingle has no CPU fallback)");
    }
    if (dist) g->device = dist->device;
    else CK(cudaGetDevice(&g->device));
    CK(cudaSetDevice(g->device));
    cudaDeviceProp prop;
    CK(cudaGetDeviceProperties(&prop, g->device));
    g->num_sms = prop.multiProcessorCount;
    if (dist && dist->stream) {
      g->stream = (cudaStream_t)dist->stream;
    } else {
      CK(cudaStreamCreateWithFlags(&g->stream, cudaStreamNonBlocking));
      g->own_stream = true;
    }
    CK(cudaStreamCreateWithFlags(&g->side, cudaStreamNonBlocking));
    // a private stream-ordered pool: freed blocks stay cached for re-runs
    // and resets, without changing the device's default pool for other users
    cudaMemPoolProps pp;
    memset(&pp, 0, sizeof pp);
    pp.allocType = cudaMemAllocationTypePinned;
    pp.handleTypes = cudaMemHandleTypeNone;
    pp.location.type = cudaMemLocationTypeDevice;
    pp.location.id = g->device;
    CK(cudaMemPoolCreate(&g->pool, &pp));
    uint64_t thr = UINT64_MAX;
    CK(cudaMemPoolSetAttribute(g->pool, cudaMemPoolAttrReleaseThreshold, &thr));
    ingest(g, n, nnz, row_ptr, rp_host, col, devptr, validate, (flags & SG_HOST_CSR) != 0);
    if (g->world > 1 || (dist && (dist->flags & SG_DIST_EXCHANGE))) {
      g->xch = exchange_create(g, dist);
      g->peer_xch = (dist->flags & SG_DIST_PEER) != 0;
    }
    sync(g);
    g->launch_base = g_launches.load();
    g->state = kCreated;
  } catch (const Fail &f) {
    st = f.st;
    t_err = g->err;
  }
  if (st != SG_OK) {
    if (g->xch) exchange_destroy(g->xch);
    if (g->stream) {
      for (DBuf *b : {&g->row_ptr, &g->col})
        if (b->p) cudaFreeAsync(b->p, g->stream);
      for (auto &c : g->cache) cudaFreeAsync(c.p, g->stream);
      cudaStreamSynchronize(g->stream);
    }
    cudaGetLastError();
    unmap_col(g);
    if (g->own_stream && g->stream) cudaStreamDestroy(g->stream);
    if (g->side) cudaStreamDestroy(g->side);
    if (g->pool) cudaMemPoolDestroy(g->pool);
    cudaGetLastError();
    return st;
  }
  *out = G.release();
  return SG_OK;
}

sg_status shingle_graph_load(sg_graph *g, int64_t n, int64_t nnz, const int64_t *row_ptr,
                             const int32_t *col, uint32_t flags) {
  return guarded(g, [&] {
    if (n < 0 || (uint64_t)n >= kP || nnz < 0 || (n > 0 && !row_ptr) || (nnz > 0 && !col))
      fail(g, SG_EINVAL, "invalid n / nnz / pointers (need 0 <= n < 2^31 - 1)");
    const bool devptr = flags & SG_DEVICE_PTRS;
    std::vector<int64_t> hrp;
    const int64_t *rp_host = row_ptr;
    if (devptr && n > 0) {
      hrp.resize((size_t)n + 1);
      CK(cudaMemcpy(hrp.data(), row_ptr, (n + 1) * 8, cudaMemcpyDeviceToHost));
      rp_host = hrp.data();
    }
    if (n > 0 && (rp_host[0] != 0 || rp_host[n] != nnz))
      fail(g, SG_EINVAL, "invalid CSR: row_ptr[0] must be 0 and row_ptr[n] must equal nnz");
    for (int l = 0; l < 2; ++l) {
      free_pass(g, g->pass[l]);
      free_groups(g, g->grp[l]);
    }
    dfree(g, g->row_ptr);
    dfree(g, g->col);
    g->e2_global = -1;
    g->ov_valid = false;
    g->state = kEmpty;                  // until the new graph is resident and valid
    ingest(g, n, nnz, row_ptr, rp_host, col, devptr, !(flags & SG_NO_VALIDATE),
           (flags & SG_HOST_CSR) != 0);
    sync(g);
    g->state = kCreated;
    g->launch_base = g_launches.load();
  }, true);
}

sg_status shingle_pass(sg_graph *g, int32_t s, int32_t c, uint64_t seed) {
  return guarded(g, [&] {
    if (s < 1 || s > kMaxS || c < 1 || c > kMaxC) fail(g, SG_EINVAL, "need 1 <= s <= 8 and 1 <= c <= 1024");
    int level;
    if (g->state == kCreated) level = 0;
    else if (g->state == kGrouped1) level = 1;
    else fail(g, SG_ESTATE, "shingle_pass: call create -> pass -> group -> pass -> group");
    if (level == 0) st_clear(g);
    PassOut &P = g->pass[level];
    free_pass(g, P);
    P.s = s;
    P.c = c;
    P.seed = seed;
    P.hA.resize((size_t)c);
    P.hB.resize((size_t)c);
    hash_pairs(seed, c, P.hA.data(), P.hB.data());
    const int st_all = level == 0 ? kStPass1 : kStPass2;
    HostMark hm;
    st_begin(g, st_all);
    st_begin(g, level == 0 ? kStSelect1 : kStSelect2);
    dalloc(g, P.A, (size_t)c * 4);
    dalloc(g, P.B, (size_t)c * 4);
    CK(cudaMemcpyAsync(P.A.p, P.hA.data(), (size_t)c * 4, cudaMemcpyHostToDevice, g->stream));
    CK(cudaMemcpyAsync(P.B.p, P.hB.data(), (size_t)c * 4, cudaMemcpyHostToDevice, g->stream));
    // ---- rows of the pass
    DBuf blk, tot;
    int64_t nrows = 0;
    if (level == 0) {
      const int64_t rows = g->row_hi - g->row_lo;
      dalloc(g, blk, (size_t)sel_scratch_elems(rows) * 8);
      dalloc(g, tot, 8);
      CK(select_csr_count(ptr<int64_t>(g->row_ptr), rows, s, ptr<int64_t>(blk), ptr<int64_t>(tot),
                          g->stream));
      CK(cudaMemcpyAsync(&nrows, tot.p, 8, cudaMemcpyDeviceToHost, g->stream));
      sync(g);
      hm("select count + sync");
      dalloc(g, P.rstart, (size_t)nrows * 8);
      dalloc(g, P.rlen, (size_t)nrows * 4);
      dalloc(g, P.rowid, (size_t)nrows * 4);
      CK(select_csr_write(ptr<int64_t>(g->row_ptr), rows, s, g->row_lo, ptr<int64_t>(blk),
                          ptr<int64_t>(P.rstart), ptr<int32_t>(P.rlen), ptr<uint32_t>(P.rowid),
                          g->stream));
      P.entries = g->col_dev;
    } else {
      Groups &G1 = g->grp[0];
      dalloc(g, blk, (size_t)sel_scratch_elems((G1.npairs + 31) / 32) * 8);
      dalloc(g, tot, 8);
      CK(select_groups_count(ptr<uint32_t>(G1.head), G1.npairs, s, ptr<int64_t>(blk),
                             ptr<int64_t>(tot), g->stream));
      CK(cudaMemcpyAsync(&nrows, tot.p, 8, cudaMemcpyDeviceToHost, g->stream));
      sync(g);
      dalloc(g, P.rstart, (size_t)nrows * 8);
      dalloc(g, P.rlen, (size_t)nrows * 4);
      CK(select_groups_write(ptr<uint32_t>(G1.head), G1.npairs, s, ptr<int64_t>(blk),
                             ptr<int64_t>(P.rstart), ptr<int32_t>(P.rlen), g->stream));
      P.entries = ptr<uint32_t>(G1.members);
      if (!g->xch && !use_group_v1() && nrows > 0) build_row_classes(g, P, nrows);
    }
    dfree(g, blk);
    dfree(g, tot);
    P.nrows = nrows;
    P.key_stride = key_stride_for(nrows);
    P.blocks = {0, nrows};
    if (level == 0) {
      g->n_e_global = g->xch ? exchange_sum(g, nrows) : nrows;
    } else if (g->xch) {
      assign_s1p_index(g, P);            // |S1'| global, canonical dense index per row
    } else {
      g->s1p_global = nrows;
      g->s1p_k0 = 0;
    }
    if (level == 1 && g->s1p_global >= (int64_t)0xFFFFFFFFll)
      fail(g, SG_EOVERFLOW, "|S1'| exceeds 2^32 - 1 (members are u32)");
    st_end(g, level == 0 ? kStSelect1 : kStSelect2);
    hm("select write enqueued");
    // ---- min-hash top-s of every row and trial (the hot kernel)
    plan_pass(g, P, level);
    hm("plan_pass");
    if (!P.deferred) {
      // SG_OVERLAP=1 (experiment, off by default): chunk 0 on the main
      // stream, the others on the side stream, overlapping the grouping of
      // earlier chunks.  Measured on gos2m: 385.4 vs 381.6 ms serialised —
      // the ALU-bound min-hash and the sort kernels contend for issue slots
      // (hist2 doubles), so the default stays serial.
      const bool overlap = g->side && g->world == 1 && P.chunks.size() > 1 && getenv("SG_OVERLAP");
      for (size_t i = 0; i < P.chunks.size(); ++i)
        compute_chunk(g, P, P.chunks[i], level == 0 ? kStHash1 : kStHash2, overlap && i > 0);
    }
    hm("min-hash enqueued");
    st_end(g, st_all);
    sync(g);
    hm("pass done (sync)");
    g->state = level == 0 ? kPassed1 : kPassed2;
  }, true);
}

sg_status group_by_shingle(sg_graph *g) {
  return guarded(g, [&] {
    int level;
    if (g->state == kPassed1) level = 0;
    else if (g->state == kPassed2) level = 1;
    else fail(g, SG_ESTATE, "group_by_shingle: needs a completed shingle_pass");
    PassOut &P = g->pass[level];
    const int c = P.c;
    st_begin(g, level == 0 ? kStGroup1 : kStGroup2);
    if (g->xch) {
      group_multi(g, level);
    } else {
      Groups &out = g->grp[level];
      free_groups(g, out);
      out.c = c;
      out.npairs = P.nrows * (int64_t)c;
      out.seg.resize((size_t)c + 1);
      for (int j = 0; j <= c; ++j) out.seg[(size_t)j] = (int64_t)j * P.nrows;
      dalloc(g, out.members, (size_t)out.npairs * 4);
      dalloc(g, out.head, (size_t)((out.npairs + 31) / 32) * 4);
      CK(cudaMemsetAsync(out.head.p, 0, out.head.bytes, g->stream));
      const uint32_t *rowid = level == 0 ? ptr<uint32_t>(P.rowid)
                                         : (P.perm.p ? ptr<uint32_t>(P.perm) : nullptr);
      const uint32_t base = level == 0 ? 0u : (uint32_t)g->s1p_k0;
      GroupScratch S;
      for (auto &ch : P.chunks) {
        if (!ch.computed) compute_chunk(g, P, ch, level == 0 ? kStHash1 : kStHash2);
        if (ch.done) {
          CK(cudaStreamWaitEvent(g->stream, ch.done, 0));   // keys computed on the side stream
          cudaEventDestroy(ch.done);
          ch.done = nullptr;
          dfree(g, ch.ctr);
        }
        std::vector<Piece> pieces;
        for (int tl = 0; tl < ch.nt; ++tl)
          pieces.push_back(Piece{tl, (int64_t)tl * P.key_stride, P.nrows, 0});
        group_any(g, ptr<uint64_t>(ch.keys), pieces, ch.t0, ch.nt, out.seg, nullptr, rowid, base,
                     out, nullptr, S, &ch.keys, level == 0 ? kStHist1 : kStHist2,
                     level == 0 ? kStScatter1 : kStScatter2, level == 0 ? kStLocal1 : kStLocal2,
                     ch.kbin.p ? ptr<uint8_t>(ch.kbin) : nullptr);
        dfree(g, ch.kbin);
        ch.computed = false;
      }
      free_scratch(g, S);
      g->pairs_global[level] = out.npairs;
    }
    st_end(g, level == 0 ? kStGroup1 : kStGroup2);
    sync(g);
    g->groups_global[level] = -1;  // computed lazily by sg_get_counts
    if (level == 1) g->e2_global = -1;
    g->state = level == 0 ? kGrouped1 : kGrouped2;
  }, true);
}

sg_status shingle_graph_reset(sg_graph *g) {
  return guarded(g, [&] {
    static const bool log = getenv("SG_ALLOC_LOG") != nullptr;
    if (log)
      fprintf(stderr, "sg alloc: pool allocations %lld, cache releases %lld, pool trims %lld, "
                      "host ms in pool calls %.2f, live %.2f GB, cached %.2f GB in %zu blocks\n",
              (long long)g->n_pool_allocs, (long long)g->n_cache_releases, (long long)g->n_trims,
              g->alloc_host_ms, g->bytes_live / 1e9, g->bytes_cached / 1e9, g->cache.size());
    g->n_pool_allocs = g->n_cache_releases = g->n_trims = 0;
    g->alloc_host_ms = 0;
    for (int l = 0; l < 2; ++l) {
      free_pass(g, g->pass[l]);
      free_groups(g, g->grp[l]);
    }
    sync(g);
    g->e2_global = -1;
    g->ov_valid = false;
    g->launch_base = g_launches.load();
    g->state = kCreated;
  });
}

void shingle_graph_destroy(sg_graph *g) {
  if (!g) return;
  cudaSetDevice(g->device);
  if (g->side) cudaStreamSynchronize(g->side);   // side-stream chunks use the buffers below
  // stream-ordered frees back into the pool (cudaFree on pool blocks leaves
  // them accounted as used), then let the pool return them to the device
  auto rel = [&](void *p) {
    if (p) cudaFreeAsync(p, g->stream);
  };
  for (int l = 0; l < 2; ++l) {
    PassOut &p = g->pass[l];
    for (DBuf *b : {&p.A, &p.B, &p.rstart, &p.rlen, &p.rowid}) rel(b->p);
    for (auto &ch : p.chunks) {
      rel(ch.keys.p);
      rel(ch.kbin.p);
      rel(ch.ctr.p);
    }
    for (DBuf *b : {&g->grp[l].members, &g->grp[l].head, &g->grp[l].okeys}) rel(b->p);
  }
  for (DBuf *b : {&g->row_ptr, &g->col}) rel(b->p);
  for (auto &c : g->cache) rel(c.p);
  if (g->side) cudaStreamSynchronize(g->side);
  if (g->stream) cudaStreamSynchronize(g->stream);
  for (cudaEvent_t e : g->ev_pool) cudaEventDestroy(e);
  for (int l = 0; l < 2; ++l)
    for (auto &ch : g->pass[l].chunks)
      if (ch.done) cudaEventDestroy(ch.done);
  if (g->xch) exchange_destroy(g->xch);
  unmap_col(g);
  if (g->own_stream && g->stream) cudaStreamDestroy(g->stream);
  if (g->side) cudaStreamDestroy(g->side);
  if (g->pool) cudaMemPoolDestroy(g->pool);
  cudaGetLastError();
  delete g;
}

sg_status sg_get_counts(const sg_graph *gc, int64_t counts[16]) {
  sg_graph *g = const_cast<sg_graph *>(gc);
  return guarded(g, [&] {
    if (!counts) fail(g, SG_EINVAL, "counts is NULL");
    const long long launches = g_launches.load() - g->launch_base;  // before getter kernels
    for (int l = 0; l < 2; ++l) {
      const bool grouped = g->state >= (l == 0 ? kGrouped1 : kGrouped2);
      if (grouped && g->groups_global[l] < 0) {
        Groups &q = g->grp[l];
        int64_t loc = device_sum_popc(g, q.head, (q.npairs + 31) / 32);
        g->groups_global[l] = g->xch ? exchange_sum(g, loc) : loc;
      }
    }
    if (g->state >= kPassed2 && g->e2_global < 0) {
      DBuf d;
      dalloc(g, d, 8);
      CK(sum_i32(ptr<int32_t>(g->pass[1].rlen), g->pass[1].nrows, ptr<unsigned long long>(d),
                 g->stream));
      unsigned long long h = 0;
      CK(cudaMemcpyAsync(&h, d.p, 8, cudaMemcpyDeviceToHost, g->stream));
      sync(g);
      dfree(g, d);
      g->e2_global = g->xch ? exchange_sum(g, (int64_t)h) : (int64_t)h;
    }
    counts[0] = g->n;
    counts[1] = g->row_lo;
    counts[2] = g->row_hi - g->row_lo;
    counts[3] = g->state >= kPassed1 ? g->n_e_global : 0;
    counts[4] = g->state >= kGrouped1 ? g->groups_global[0] : 0;
    counts[5] = g->state >= kPassed2 ? g->s1p_global : 0;
    counts[6] = g->state >= kGrouped2 ? g->groups_global[1] : 0;
    counts[7] = g->state >= kGrouped1 ? g->pairs_global[0] : 0;
    counts[8] = g->state >= kGrouped2 ? g->pairs_global[1] : 0;
    counts[9] = g->state;
    counts[10] = g->state >= kPassed2 ? g->e2_global : 0;
    counts[11] = (int64_t)launches;
    for (int l = 0; l < 2; ++l) {
      const PassOut &P = g->pass[l];
      const int64_t nch = (int64_t)P.chunks.size();
      counts[12 + l] = P.deferred ? -nch : nch;
    }
    counts[14] = g->world;                    // ranks of the exchange (communicator size)
    counts[15] = g->xch ? 1 : 0;              // owner-routed exchange path on
  }, true);
}

sg_status sg_get_shingles_range(sg_graph *g, int32_t level, int32_t t0, int32_t t1, uint64_t *ids,
                                uint32_t *rowid, int64_t cap_rows, int64_t *rows, int32_t *c) {
  return guarded(g, [&] {
    if (level != 1 && level != 2) fail(g, SG_EINVAL, "level must be 1 or 2");
    const int l = level - 1;
    if (g->state < (l == 0 ? kPassed1 : kPassed2)) fail(g, SG_ESTATE, "pass not run yet");
    PassOut &P = g->pass[l];
    if (t1 < 0) t1 = P.c;
    if (t0 < 0 || t0 > t1 || t1 > P.c) fail(g, SG_EINVAL, "need 0 <= t0 <= t1 <= c");
    if (rows) *rows = P.nrows;
    if (c) *c = P.c;
    if (!ids && !rowid) return;
    if (cap_rows < P.nrows) fail(g, SG_EINVAL, "buffer too small");
    if (ids) {
      const int nt = t1 - t0;
      std::vector<int64_t> rq((size_t)(P.nrows * nt));
      std::vector<int32_t> tq(rq.size());
      for (int64_t r = 0; r < P.nrows; ++r)
        for (int j = 0; j < nt; ++j) {
          rq[(size_t)(r * nt + j)] = r;
          tq[(size_t)(r * nt + j)] = t0 + j;
        }
      std::vector<uint64_t> v = recompute_ids(g, l, rq, tq);
      if (!v.empty()) memcpy(ids, v.data(), v.size() * 8);
    }
    if (rowid) {
      if (l == 0) {
        if (P.nrows) {
          CK(cudaMemcpyAsync(rowid, P.rowid.p, (size_t)P.nrows * 4, cudaMemcpyDeviceToHost, g->stream));
          sync(g);
        }
      } else {
        if (P.rowid.p && P.nrows) {           // multi-rank: canonical k of each row
          CK(cudaMemcpyAsync(rowid, P.rowid.p, (size_t)P.nrows * 4, cudaMemcpyDeviceToHost,
                             g->stream));
          sync(g);
        } else {
          for (int64_t r = 0; r < P.nrows; ++r) rowid[r] = (uint32_t)(g->s1p_k0 + r);
        }
      }
    }
  });
}

sg_status sg_get_shingles(sg_graph *g, int32_t level, uint64_t *ids, uint32_t *rowid,
                          int64_t cap_rows, int64_t *rows, int32_t *c) {
  return sg_get_shingles_range(g, level, 0, -1, ids, rowid, cap_rows, rows, c);
}

sg_status sg_get_groups_range(sg_graph *g, int32_t level, int32_t t0, int32_t t1,
                              int64_t *trial_goffs, uint64_t *ids, int64_t *offs, uint32_t *members,
                              const int64_t caps[2], int64_t counts[3]) {
  return guarded(g, [&] {
    if (level != 1 && level != 2) fail(g, SG_EINVAL, "level must be 1 or 2");
    const int l = level - 1;
    if (g->state < (l == 0 ? kGrouped1 : kGrouped2)) fail(g, SG_ESTATE, "not grouped yet");
    const int c = g->grp[l].c;
    if (t1 < 0) t1 = c;
    if (t0 < 0 || t0 > t1 || t1 > c) fail(g, SG_EINVAL, "need 0 <= t0 <= t1 <= c");
    HostGroups H;
    const bool fill = trial_goffs || ids || offs || members;
    host_groups(g, l, H, fill && ids != nullptr, t0, t1);
    const int64_t G = (int64_t)H.offs.size() - 1;
    if (counts) {
      counts[0] = G;
      counts[1] = (int64_t)H.members.size();
      counts[2] = t1 - t0;
    }
    if (!fill) return;
    if (!caps || caps[0] < G || caps[1] < (int64_t)H.members.size())
      fail(g, SG_EINVAL, "buffers too small");
    if (trial_goffs) memcpy(trial_goffs, H.trial_goffs.data(), H.trial_goffs.size() * 8);
    if (ids && G) memcpy(ids, H.ids.data(), H.ids.size() * 8);
    if (offs) memcpy(offs, H.offs.data(), H.offs.size() * 8);
    if (members && !H.members.empty()) memcpy(members, H.members.data(), H.members.size() * 4);
  });
}

sg_status sg_get_groups(sg_graph *g, int32_t level, int64_t *trial_goffs, uint64_t *ids,
                        int64_t *offs, uint32_t *members, const int64_t caps[2], int64_t counts[3]) {
  return sg_get_groups_range(g, level, 0, -1, trial_goffs, ids, offs, members, caps, counts);
}

sg_status sg_get_s1p(sg_graph *g, int64_t *s1p_group, int64_t cap, int64_t *count, int64_t *k0) {
  return guarded(g, [&] {
    if (g->state < kPassed2) fail(g, SG_ESTATE, "pass II not run yet");
    PassOut &P = g->pass[1];
    if (count) *count = P.nrows;
    if (k0) *k0 = g->s1p_k0;
    if (!s1p_group) return;
    if (cap < P.nrows) fail(g, SG_EINVAL, "buffer too small");
    std::vector<int64_t> rs = d2h<int64_t>(g, P.rstart, (size_t)P.nrows);
    Groups &q = g->grp[0];
    std::vector<uint32_t> head = d2h<uint32_t>(g, q.head, (size_t)((q.npairs + 31) / 32));
    // group index of the group starting at pair rs[k] = heads before rs[k]
    int64_t gi = -1, k = 0;
    for (int64_t i = 0; i < q.npairs && k < P.nrows; ++i) {
      if ((head[(size_t)(i >> 5)] >> (i & 31)) & 1u) ++gi;
      while (k < P.nrows && rs[(size_t)k] == i) s1p_group[k++] = gi;
    }
  });
}

sg_status sg_get_hash_params(sg_graph *g, int32_t level, uint32_t *A, uint32_t *B, int32_t cap) {
  return guarded(g, [&] {
    if (level != 1 && level != 2) fail(g, SG_EINVAL, "level must be 1 or 2");
    PassOut &P = g->pass[level - 1];
    if (P.c == 0) fail(g, SG_ESTATE, "pass not run yet");
    if (cap < P.c) fail(g, SG_EINVAL, "buffer too small");
    if (A) memcpy(A, P.hA.data(), (size_t)P.c * 4);
    if (B) memcpy(B, P.hB.data(), (size_t)P.c * 4);
  });
}

sg_status sg_get_stage_ms(const sg_graph *gc, float *ms, int32_t cap, int32_t *n) {
  sg_graph *g = const_cast<sg_graph *>(gc);
  return guarded(g, [&] {
    const int k = std::min<int>(cap, kNumStages);
    if (ms) sync(g);
    for (int i = 0; i < k; ++i) {
      float tot = 0.f;
      if (ms) {
        for (auto &pr : g->st[i]) {
          if (pr.second < 0) continue;
          float v = 0.f;
          if (cudaEventElapsedTime(&v, g->ev_pool[(size_t)pr.first], g->ev_pool[(size_t)pr.second]) ==
              cudaSuccess)
            tot += v;
          else
            cudaGetLastError();
        }
        ms[i] = tot;
      }
    }
    if (n) *n = k;
  });
}

sg_status report_dense_subgraphs(sg_graph *g, int32_t mode, int32_t min_size, int32_t *labels,
                                 int64_t *n_clusters) {
  return guarded(g, [&] {
    const bool host = (mode & SG_REPORT_HOST) != 0;
    mode &= ~SG_REPORT_HOST;
    if (mode != 0 && mode != 1) fail(g, SG_EINVAL, "mode must be 0 or 1 (| SG_REPORT_HOST)");
    if (g->state != kGrouped2) fail(g, SG_ESTATE, "report needs both passes grouped");
    if (g->world > 1) require_single(g, "report_dense_subgraphs");
    PassOut &P1 = g->pass[0];
    PassOut &P2 = g->pass[1];
    if (!host) {
      // ---- device union-find (kernels_report.cu)
      ReportArgs a;
      a.n = g->n;
      a.mode = mode;
      a.min_size = min_size;
      a.s1 = P1.s;
      a.s2 = P2.s;
      a.A1 = ptr<uint32_t>(P1.A);
      a.B1 = ptr<uint32_t>(P1.B);
      a.A2 = ptr<uint32_t>(P2.A);
      a.B2 = ptr<uint32_t>(P2.B);
      a.row_ptr = ptr<int64_t>(g->row_ptr);
      a.col = g->col_dev;
      a.members1 = ptr<uint32_t>(g->grp[0].members);
      a.rows1 = P1.nrows;
      a.rstart2 = ptr<int64_t>(P2.rstart);
      a.rlen2 = ptr<int32_t>(P2.rlen);
      a.nk = P2.nrows;
      a.members2 = ptr<uint32_t>(g->grp[1].members);
      a.head2 = ptr<uint32_t>(g->grp[1].head);
      a.npairs2 = g->grp[1].npairs;
      a.rows2 = P2.nrows;
      // mode 0, s2 <= 2: the S1' nodes in length-class order for the per-node
      // second-level constituents (built here unless pass II kept them)
      PassOut tmp;
      const bool nodes = mode == 0 && P2.s <= 2 && P2.nrows > 0;
      PassOut *pc = nullptr;
      if (nodes) {
        if (P2.perm.p) {
          pc = &P2;
        } else {
          tmp.rstart = P2.rstart;                 // borrowed (not freed through tmp)
          tmp.rlen = P2.rlen;
          build_row_classes(g, tmp, P2.nrows);
          pc = &tmp;
        }
        a.perm2 = ptr<uint32_t>(pc->perm);
        a.rstart2p = ptr<int64_t>(pc->rstart_p);
        a.rlen2p = ptr<int32_t>(pc->rlen_p);
        a.nshort2 = pc->n_split;
        a.c2 = P2.c;
      }
      DBuf parent, rep1, size, dlab, dnc;
      dalloc(g, parent, (size_t)a.n * 4);
      dalloc(g, rep1, (size_t)a.nk * 4);
      dalloc(g, size, (size_t)a.n * 4);
      dalloc(g, dlab, (size_t)a.n * 4);
      dalloc(g, dnc, 8);
      g->st[kStReport].clear();
      st_begin(g, kStReport);
      CK(report_device(a, ptr<uint32_t>(parent), ptr<uint32_t>(rep1), ptr<uint32_t>(size),
                       ptr<int32_t>(dlab), ptr<unsigned long long>(dnc), g->num_sms, g->stream));
      st_end(g, kStReport);
      unsigned long long nc = 0;
      if (labels)
        CK(cudaMemcpyAsync(labels, dlab.p, (size_t)a.n * 4, cudaMemcpyDeviceToHost, g->stream));
      CK(cudaMemcpyAsync(&nc, dnc.p, 8, cudaMemcpyDeviceToHost, g->stream));
      sync(g);
      for (DBuf *b : {&parent, &rep1, &size, &dlab, &dnc}) dfree(g, *b);
      if (pc == &tmp) {
        for (DBuf *b : {&tmp.perm, &tmp.rstart_p, &tmp.rlen_p}) dfree(g, *b);
        tmp.rstart = DBuf();
        tmp.rlen = DBuf();
      }
      if (n_clusters) *n_clusters = (int64_t)nc;
      return;
    }
    HostGroups H1, H2;
    host_groups(g, 0, H1, true);
    host_groups(g, 1, H2, mode == 0);
    // S1' nodes: pass-II rows, in order; the group of row k starts at rstart[k]
    std::vector<int64_t> rs = d2h<int64_t>(g, P2.rstart, (size_t)P2.nrows);
    std::vector<int32_t> rl = d2h<int32_t>(g, P2.rlen, (size_t)P2.nrows);
    const int64_t nk = P2.nrows;
    std::vector<int32_t> trial1((size_t)nk);
    std::vector<uint64_t> id1((size_t)nk);
    std::vector<int64_t> lo2((size_t)nk + 1, 0);
    std::vector<uint32_t> lm;
    {
      size_t gi = 0;
      int j = 0;
      for (int64_t k = 0; k < nk; ++k) {
        while (H1.offs[gi] < rs[(size_t)k]) ++gi;
        while (g->grp[0].seg[(size_t)j + 1] <= rs[(size_t)k]) ++j;
        trial1[(size_t)k] = j;
        id1[(size_t)k] = H1.ids[gi];
        lo2[(size_t)k] = (int64_t)lm.size();
        lm.insert(lm.end(), H1.members.begin() + rs[(size_t)k],
                  H1.members.begin() + rs[(size_t)k] + rl[(size_t)k]);
      }
      lo2[(size_t)nk] = (int64_t)lm.size();
    }
    const int64_t nh = (int64_t)H2.offs.size() - 1;
    std::vector<int32_t> trial2((size_t)nh);
    for (int t = 0; t < g->grp[1].c; ++t)
      for (int64_t h = H2.trial_goffs[(size_t)t]; h < H2.trial_goffs[(size_t)t + 1]; ++h)
        trial2[(size_t)h] = t;
    std::vector<int64_t> hrp;
    std::vector<int32_t> hcol;
    if (P1.s >= 3 && mode == 0) {
      hrp = d2h<int64_t>(g, g->row_ptr, (size_t)(g->row_hi - g->row_lo + 1));
      hcol.resize((size_t)g->nnz_local);
      if (g->nnz_local) {
        CK(cudaMemcpyAsync(hcol.data(), g->col_dev, (size_t)g->nnz_local * 4, cudaMemcpyDefault, g->stream));
        sync(g);
      }
    }
    ReportInput in;
    in.n = g->n;
    in.s1 = P1.s;
    in.s2 = P2.s;
    in.A1 = P1.hA.data();
    in.B1 = P1.hB.data();
    in.A2 = P2.hA.data();
    in.B2 = P2.hB.data();
    in.nk = nk;
    in.trial1 = trial1.data();
    in.id1 = id1.data();
    in.loff = lo2.data();
    in.lmem = lm.data();
    in.nh = nh;
    in.trial2 = trial2.data();
    in.id2 = H2.ids.empty() ? nullptr : H2.ids.data();
    in.koff = H2.offs.data();
    in.kmem = H2.members.data();
    in.row_ptr = hrp.empty() ? nullptr : hrp.data();
    in.col = hcol.empty() ? nullptr : hcol.data();
    const int64_t nc = report_host(in, mode, min_size, labels);
    if (n_clusters) *n_clusters = nc;
  });
}

static void overlap_compute(sg_graph *g, int32_t mode, int32_t min_size) {
    PassOut &P1 = g->pass[0];
    PassOut &P2 = g->pass[1];
    ReportArgs a;
    a.n = g->n;
    a.mode = mode;
    a.min_size = min_size;
    a.s1 = P1.s;
    a.s2 = P2.s;
    a.A1 = ptr<uint32_t>(P1.A);
    a.B1 = ptr<uint32_t>(P1.B);
    a.row_ptr = ptr<int64_t>(g->row_ptr);
    a.col = g->col_dev;
    a.members1 = ptr<uint32_t>(g->grp[0].members);
    a.rows1 = P1.nrows;
    a.rstart2 = ptr<int64_t>(P2.rstart);
    a.rlen2 = ptr<int32_t>(P2.rlen);
    a.nk = P2.nrows;
    a.members2 = ptr<uint32_t>(g->grp[1].members);
    a.head2 = ptr<uint32_t>(g->grp[1].head);
    a.npairs2 = g->grp[1].npairs;
    a.rows2 = P2.nrows;
    DBuf parentK, eoff, keys, sorted, temp, dn;
    dalloc(g, dn, 8);
    int64_t nkeys = a.nk * (int64_t)a.s1;
    if (mode == 1) {
      unsigned long long e2 = 0;
      CK(sum_i32(a.rlen2, a.nk, ptr<unsigned long long>(dn), g->stream));
      CK(cudaMemcpyAsync(&e2, dn.p, 8, cudaMemcpyDeviceToHost, g->stream));
      sync(g);
      nkeys = (int64_t)e2;
    }
    if (nkeys > INT32_MAX || a.nk > INT32_MAX)
      fail(g, SG_EOVERFLOW, "report_overlapping_clusters: more than 2^31 constituents");
    const size_t tb = overlap_temp_bytes(a.nk, nkeys);
    dalloc(g, parentK, (size_t)a.nk * 4);
    dalloc(g, eoff, (size_t)a.nk * 8);
    dalloc(g, keys, (size_t)nkeys * 8);
    dalloc(g, sorted, (size_t)nkeys * 8);
    dalloc(g, temp, tb);
    CK(overlap_device(a, ptr<uint32_t>(parentK), ptr<int64_t>(eoff), ptr<uint64_t>(keys),
                      ptr<uint64_t>(sorted), nkeys, temp.p, temp.bytes, ptr<int64_t>(dn),
                      g->num_sms, g->stream));
    int64_t nu = 0;
    CK(cudaMemcpyAsync(&nu, dn.p, 8, cudaMemcpyDeviceToHost, g->stream));
    sync(g);
    std::vector<uint64_t> u((size_t)nu);
    if (nu) CK(cudaMemcpyAsync(u.data(), keys.p, (size_t)nu * 8, cudaMemcpyDeviceToHost, g->stream));
    sync(g);
    for (DBuf *b : {&parentK, &eoff, &keys, &sorted, &temp, &dn}) dfree(g, *b);
    if (nu && u[(size_t)nu - 1] == ~0ull) --nu;         // rows shorter than s1 (none in practice)
    // split the sorted (root, vertex) list into clusters; drop the small ones
    const int64_t thr = std::max<int32_t>(1, min_size);
    g->ov_offs.assign(1, 0);
    g->ov_verts.clear();
    g->ov_verts.reserve((size_t)nu);
    for (int64_t i = 0; i < nu;) {
      int64_t e = i + 1;
      while (e < nu && (u[(size_t)e] >> 32) == (u[(size_t)i] >> 32)) ++e;
      if (e - i >= thr) {
        for (int64_t x = i; x < e; ++x) g->ov_verts.push_back((uint32_t)u[(size_t)x]);
        g->ov_offs.push_back((int64_t)g->ov_verts.size());
      }
      i = e;
    }
}

sg_status report_overlapping_clusters(sg_graph *g, int32_t mode, int32_t min_size, int64_t *offs,
                                      uint32_t *verts, const int64_t caps[2], int64_t counts[2]) {
  return guarded(g, [&] {
    if (mode != 0 && mode != 1) fail(g, SG_EINVAL, "mode must be 0 or 1");
    if (!counts) fail(g, SG_EINVAL, "counts is NULL");
    if (g->state != kGrouped2) fail(g, SG_ESTATE, "report needs both passes grouped");
    if (g->world > 1) require_single(g, "report_overlapping_clusters");
    if (!(g->ov_valid && g->ov_mode == mode && g->ov_min == min_size)) {
      overlap_compute(g, mode, min_size);
      g->ov_valid = true;
      g->ov_mode = mode;
      g->ov_min = min_size;
    }
    const int64_t nc = (int64_t)g->ov_offs.size() - 1, nv = (int64_t)g->ov_verts.size();
    if (offs || verts) {
      if (!caps || caps[0] < nc + 1 || caps[1] < nv) fail(g, SG_EINVAL, "buffers too small");
      if (offs) std::copy(g->ov_offs.begin(), g->ov_offs.end(), offs);
      if (verts) std::copy(g->ov_verts.begin(), g->ov_verts.end(), verts);
      g->ov_valid = false;                              // filled: release the host copy
      std::vector<int64_t>().swap(g->ov_offs);
      std::vector<uint32_t>().swap(g->ov_verts);
    }
    counts[0] = nc;
    counts[1] = nv;
  });
}

sg_status sg_cluster_density(sg_graph *g, const int32_t *labels, int32_t min_size, double *mean,
                             double *stddev, int64_t *n_clusters) {
  return guarded(g, [&] {
    if (!labels) fail(g, SG_EINVAL, "labels is NULL");
    if (g->world > 1) require_single(g, "sg_cluster_density");
    if (g->state < kCreated) fail(g, SG_ESTATE, "no graph");
    const int64_t n = g->n;
    for (int64_t v = 0; v < n; ++v)
      if (labels[v] < 0 || labels[v] >= n) fail(g, SG_EINVAL, "labels must lie in [0, n)");
    DBuf dl, de, ds;
    dalloc(g, dl, (size_t)n * 4);
    dalloc(g, de, (size_t)n * 8);
    dalloc(g, ds, (size_t)n * 4);
    CK(cudaMemcpyAsync(dl.p, labels, (size_t)n * 4, cudaMemcpyHostToDevice, g->stream));
    CK(density_device(ptr<int64_t>(g->row_ptr), g->col_dev, n, ptr<int32_t>(dl),
                      ptr<unsigned long long>(de), ptr<uint32_t>(ds), g->num_sms, g->stream));
    std::vector<unsigned long long> e2((size_t)n);
    std::vector<uint32_t> sz((size_t)n);
    CK(cudaMemcpyAsync(e2.data(), de.p, (size_t)n * 8, cudaMemcpyDeviceToHost, g->stream));
    CK(cudaMemcpyAsync(sz.data(), ds.p, (size_t)n * 4, cudaMemcpyDeviceToHost, g->stream));
    sync(g);
    for (DBuf *b : {&dl, &de, &ds}) dfree(g, *b);
    // mean and population standard deviation over clusters of >= max(2, min_size)
    const int64_t thr = std::max<int32_t>(2, min_size);
    int64_t c = 0;
    double s1 = 0.0, s2 = 0.0;
    for (int64_t r = 0; r < n; ++r) {
      const int64_t k = sz[(size_t)r];
      if (k < thr) continue;
      // each stored entry (u, v), u != v, inside the cluster is half an edge
      // (symmetric rows: exactly the edge count; AMB-21)
      const double d = ((double)e2[(size_t)r] / 2.0) / ((double)k * (double)(k - 1) / 2.0);
      ++c;
      s1 += d;
      s2 += d * d;
    }
    const double mu = c ? s1 / (double)c : 0.0;
    if (mean) *mean = mu;
    if (stddev) *stddev = c ? std::sqrt(std::max(0.0, s2 / (double)c - mu * mu)) : 0.0;
    if (n_clusters) *n_clusters = c;
  });
}

sg_status sg_partition_agreement(sg_graph *g, const int32_t *test_labels,
                                 const int32_t *bench_labels, int64_t counts[4]) {
  return guarded(g, [&] {
    if (!test_labels || !bench_labels || !counts) fail(g, SG_EINVAL, "NULL argument");
    if (g->world > 1) require_single(g, "sg_partition_agreement");
    const int64_t n = g->n;
    if (n > INT32_MAX) fail(g, SG_EOVERFLOW, "n > 2^31");
    for (int64_t v = 0; v < n; ++v)
      if (test_labels[v] < 0 || test_labels[v] >= n || bench_labels[v] < 0 || bench_labels[v] >= n)
        fail(g, SG_EINVAL, "labels must lie in [0, n)");
    const size_t tb = agreement_temp_bytes(n);
    DBuf dt, db, ct, cb, cj, k1, k2, temp, runs, out;
    dalloc(g, dt, (size_t)n * 4);
    dalloc(g, db, (size_t)n * 4);
    dalloc(g, ct, (size_t)n * 4);
    dalloc(g, cb, (size_t)n * 4);
    dalloc(g, cj, (size_t)n * 4);
    dalloc(g, k1, (size_t)n * 8);
    dalloc(g, k2, (size_t)n * 8);
    dalloc(g, temp, tb);
    dalloc(g, runs, 8);
    dalloc(g, out, 24);
    CK(cudaMemcpyAsync(dt.p, test_labels, (size_t)n * 4, cudaMemcpyHostToDevice, g->stream));
    CK(cudaMemcpyAsync(db.p, bench_labels, (size_t)n * 4, cudaMemcpyHostToDevice, g->stream));
    CK(agreement_device(ptr<int32_t>(dt), ptr<int32_t>(db), n, ptr<uint32_t>(ct),
                        ptr<uint32_t>(cb), ptr<uint32_t>(cj), ptr<uint64_t>(k1), ptr<uint64_t>(k2),
                        temp.p, temp.bytes, ptr<int64_t>(runs), ptr<unsigned long long>(out),
                        g->num_sms, g->stream));
    unsigned long long h[3] = {0, 0, 0};
    CK(cudaMemcpyAsync(h, out.p, 24, cudaMemcpyDeviceToHost, g->stream));
    sync(g);
    for (DBuf *b : {&dt, &db, &ct, &cb, &cj, &k1, &k2, &temp, &runs, &out}) dfree(g, *b);
    const unsigned long long all = (unsigned long long)n * (unsigned long long)(n > 0 ? n - 1 : 0) / 2;
    counts[0] = (int64_t)h[0];                          // TP: together in both
    counts[1] = (int64_t)(h[1] - h[0]);                 // FP: together in test only
    counts[2] = (int64_t)(h[2] - h[0]);                 // FN: together in benchmark only
    counts[3] = (int64_t)(all - h[1] - h[2] + h[0]);    // TN: apart in both
  });
}

sg_status sg_connected_components(sg_graph *g, int32_t *labels, int64_t *n_components) {
  return guarded(g, [&] {
    if (!labels) fail(g, SG_EINVAL, "labels is NULL");
    if (g->world > 1) require_single(g, "sg_connected_components");
    const int64_t n = g->n;
    DBuf parent, dl;
    dalloc(g, parent, (size_t)n * 4);
    dalloc(g, dl, (size_t)n * 4);
    CK(components_device(ptr<int64_t>(g->row_ptr), g->col_dev, n,
                         ptr<uint32_t>(parent), ptr<int32_t>(dl), g->num_sms, g->stream));
    if (n) CK(cudaMemcpyAsync(labels, dl.p, (size_t)n * 4, cudaMemcpyDeviceToHost, g->stream));
    sync(g);
    dfree(g, parent);
    dfree(g, dl);
    if (n_components) {
      int64_t c = 0;
      for (int64_t v = 0; v < n; ++v) c += labels[v] == (int32_t)v;
      *n_components = c;
    }
  });
}

}  // extern "C"
