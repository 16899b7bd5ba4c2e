// exchange.cu — multi-GPU transport: NCCL (dlopen) or in-process loopback.
#include <dlfcn.h>
#include <nccl.h>

#include <chrono>
#include <condition_variable>
#include <cstdlib>
#include <cstring>
#include <thread>
#include <mutex>
#include <vector>

#include "exchange.h"

// ---------------------------------------------------------------- loopback
struct sg_loopback {
  int world = 1;
  std::mutex mu;
  std::condition_variable cv;
  int arrived = 0;
  uint64_t gen = 0;
  std::vector<std::vector<int64_t>> hv;   // published host vectors
  std::vector<const void *> dptr;         // published device send buffers
  std::vector<const int64_t *> doff;      // their element offsets (host)
  bool broken = false;

  // false if a peer aborted (the group is unusable afterwards)
  bool barrier() {
    std::unique_lock<std::mutex> lk(mu);
    if (broken) return false;
    const uint64_t my = gen;
    if (++arrived == world) {
      arrived = 0;
      ++gen;
      cv.notify_all();
    } else {
      cv.wait(lk, [&] { return gen != my || broken; });
    }
    return !broken;
  }
  void abort() {
    std::lock_guard<std::mutex> lk(mu);
    broken = true;
    cv.notify_all();
  }
};

namespace sg {

namespace {

// NCCL entry points resolved at run time
struct NcclApi {
  void *so = nullptr;
  decltype(&ncclGetUniqueId) getUniqueId = nullptr;
  decltype(&ncclCommInitRank) commInitRank = nullptr;
  decltype(&ncclCommDestroy) commDestroy = nullptr;
  decltype(&ncclAllGather) allGather = nullptr;
  decltype(&ncclSend) send = nullptr;
  decltype(&ncclRecv) recv = nullptr;
  decltype(&ncclGroupStart) groupStart = nullptr;
  decltype(&ncclGroupEnd) groupEnd = nullptr;
  decltype(&ncclGetErrorString) errStr = nullptr;
  decltype(&ncclCommGetAsyncError) asyncError = nullptr;   // optional (polling)
  decltype(&ncclCommAbort) commAbort = nullptr;            // optional (polling)
};

NcclApi *nccl_api(std::string *why) {
  static NcclApi api;
  static bool tried = false, ok = false;
  static std::mutex m;
  std::lock_guard<std::mutex> lk(m);
  if (!tried) {
    tried = true;
    for (const char *name : {"libnccl.so.2", "libnccl.so"}) {
      api.so = dlopen(name, RTLD_NOW | RTLD_GLOBAL);
      if (api.so) break;
    }
    if (api.so) {
      api.getUniqueId = (decltype(api.getUniqueId))dlsym(api.so, "ncclGetUniqueId");
      api.commInitRank = (decltype(api.commInitRank))dlsym(api.so, "ncclCommInitRank");
      api.commDestroy = (decltype(api.commDestroy))dlsym(api.so, "ncclCommDestroy");
      api.allGather = (decltype(api.allGather))dlsym(api.so, "ncclAllGather");
      api.send = (decltype(api.send))dlsym(api.so, "ncclSend");
      api.recv = (decltype(api.recv))dlsym(api.so, "ncclRecv");
      api.groupStart = (decltype(api.groupStart))dlsym(api.so, "ncclGroupStart");
      api.groupEnd = (decltype(api.groupEnd))dlsym(api.so, "ncclGroupEnd");
      api.errStr = (decltype(api.errStr))dlsym(api.so, "ncclGetErrorString");
      api.asyncError = (decltype(api.asyncError))dlsym(api.so, "ncclCommGetAsyncError");
      api.commAbort = (decltype(api.commAbort))dlsym(api.so, "ncclCommAbort");
      ok = api.getUniqueId && api.commInitRank && api.commDestroy && api.allGather && api.send &&
           api.recv && api.groupStart && api.groupEnd && api.errStr;
    }
  }
  if (!ok && why) *why = api.so ? "libnccl.so.2 lacks required symbols" : "libnccl.so.2 not found";
  return ok ? &api : nullptr;
}

}  // namespace

struct Exchange {
  int rank = 0, world = 1;
  sg_loopback *lb = nullptr;
  NcclApi *nccl = nullptr;
  ncclComm_t comm = nullptr;
  void *dbuf = nullptr;      // device scratch for NCCL all-gathers
  size_t dbytes = 0;
};

// Wait for the handle's stream while polling the communicator: a peer that
// failed (or a broken link) surfaces as an asynchronous NCCL error; the
// communicator is then aborted so this rank returns SG_ENCCL instead of
// hanging in a collective.  SG_NCCL_TIMEOUT_S (default 600) bounds the wait.
static void nccl_wait(sg_graph *g, const char *what) {
  Exchange *x = g->xch;
  static const double limit = [] {
    const char *e = getenv("SG_NCCL_TIMEOUT_S");
    return e ? atof(e) : 600.0;
  }();
  const auto t0 = std::chrono::steady_clock::now();
  for (int it = 0;; ++it) {
    const cudaError_t q = cudaStreamQuery(g->stream);
    if (q == cudaSuccess) return;
    if (q != cudaErrorNotReady) ck(g, q, what);
    if (x->nccl->asyncError) {
      ncclResult_t ae = ncclSuccess;
      if (x->nccl->asyncError(x->comm, &ae) == ncclSuccess && ae != ncclSuccess && ae != ncclInProgress) {
        if (x->nccl->commAbort) x->nccl->commAbort(x->comm);
        x->comm = nullptr;
        fail(g, SG_ENCCL, std::string(what) + ": asynchronous NCCL error: " + x->nccl->errStr(ae));
      }
    }
    if (it > 2000) {
      std::this_thread::sleep_for(std::chrono::microseconds(50));
      const double el = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
      if (el > limit) {
        if (x->nccl->commAbort) x->nccl->commAbort(x->comm);
        x->comm = nullptr;
        fail(g, SG_ENCCL, std::string(what) + ": timed out (SG_NCCL_TIMEOUT_S); communicator aborted");
      }
    }
  }
}

static void nck(sg_graph *g, ncclResult_t r, const char *what) {
  if (r != ncclSuccess) {
    Exchange *x = g->xch;
    fail(g, SG_ENCCL, std::string(what) + ": " + (x && x->nccl ? x->nccl->errStr(r) : "nccl error"));
  }
}

Exchange *exchange_create(sg_graph *g, const sg_dist *d) {
  Exchange *x = new Exchange();
  x->rank = d->rank;
  x->world = d->world;
  if (d->loopback) {
    x->lb = reinterpret_cast<sg_loopback *>(d->loopback);
    if (x->lb->world != d->world) {
      delete x;
      fail(g, SG_EINVAL, "loopback group size differs from sg_dist.world");
    }
    return x;
  }
  std::string why;
  x->nccl = nccl_api(&why);
  if (!x->nccl) {
    delete x;
    fail(g, SG_ENCCL, "world > 1 needs NCCL: " + why);
  }
  if (!d->nccl_uid) {
    delete x;
    fail(g, SG_EINVAL, "world > 1 needs sg_dist.nccl_uid (or a loopback group)");
  }
  ncclUniqueId uid;
  memcpy(&uid, d->nccl_uid, sizeof(uid));
  g->xch = x;
  nck(g, x->nccl->commInitRank(&x->comm, d->world, uid, d->rank), "ncclCommInitRank");
  return x;
}

static void lb_barrier(sg_graph *g, sg_loopback *lb) {
  if (!lb->barrier()) fail(g, SG_ESTATE, "a peer rank of the loopback group failed");
}

void exchange_abort(Exchange *x) {
  if (x && x->lb) x->lb->abort();
}

void exchange_destroy(Exchange *x) {
  if (!x) return;
  if (x->comm && x->nccl) x->nccl->commDestroy(x->comm);
  if (x->dbuf) cudaFree(x->dbuf);
  delete x;
}

void x_allgather_i64(sg_graph *g, const int64_t *mine, int64_t n, int64_t *all) {
  Exchange *x = g->xch;
  if (x->lb) {
    sg_loopback *lb = x->lb;
    lb->hv[(size_t)x->rank].assign(mine, mine + n);
    lb_barrier(g, lb);
    for (int r = 0; r < x->world; ++r)
      memcpy(all + (int64_t)r * n, lb->hv[(size_t)r].data(), (size_t)n * 8);
    lb_barrier(g, lb);
    return;
  }
  const size_t need = (size_t)n * 8 * (size_t)(x->world + 1);
  if (x->dbytes < need) {
    if (x->dbuf) cudaFree(x->dbuf);
    ck(g, cudaMalloc(&x->dbuf, need), "cudaMalloc (exchange)");
    x->dbytes = need;
  }
  int64_t *din = reinterpret_cast<int64_t *>(x->dbuf);
  int64_t *dout = din + n;
  ck(g, cudaMemcpyAsync(din, mine, (size_t)n * 8, cudaMemcpyHostToDevice, g->stream), "H2D");
  if (!x->comm) fail(g, SG_ENCCL, "communicator was aborted");
  nck(g, x->nccl->allGather(din, dout, (size_t)n, ncclInt64, x->comm, g->stream), "ncclAllGather");
  ck(g, cudaMemcpyAsync(all, dout, (size_t)n * 8 * x->world, cudaMemcpyDeviceToHost, g->stream), "D2H");
  nccl_wait(g, "ncclAllGather");
}

int64_t exchange_sum(sg_graph *g, int64_t v) {
  std::vector<int64_t> all((size_t)g->world);
  x_allgather_i64(g, &v, 1, all.data());
  int64_t s = 0;
  for (int64_t a : all) s += a;
  return s;
}

int64_t exchange_min(sg_graph *g, int64_t v) {
  std::vector<int64_t> all((size_t)g->world);
  x_allgather_i64(g, &v, 1, all.data());
  int64_t s = all[0];
  for (int64_t a : all) s = a < s ? a : s;
  return s;
}

void x_alltoallv2(sg_graph *g, const void *send1, void *recv1, size_t eb1, const void *send2,
                  void *recv2, size_t eb2, const int64_t *soff, const int64_t *roff) {
  Exchange *x = g->xch;
  const int R = x->world, me = x->rank;
  if (x->lb) {
    sg_loopback *lb = x->lb;
    ck(g, cudaStreamSynchronize(g->stream), "sync");     // send data complete
    for (int pass = 0; pass < 2; ++pass) {
      const void *send = pass ? send2 : send1;
      void *recv = pass ? recv2 : recv1;
      const size_t eb = pass ? eb2 : eb1;
      if (!send) continue;
      lb->dptr[(size_t)me] = send;
      lb->doff[(size_t)me] = soff;
      lb_barrier(g, lb);
      for (int s = 0; s < R; ++s) {
        const int64_t a = lb->doff[(size_t)s][me], b = lb->doff[(size_t)s][me + 1];
        if (b > a)
          ck(g, cudaMemcpyAsync((char *)recv + roff[s] * eb,
                                (const char *)lb->dptr[(size_t)s] + a * eb, (size_t)(b - a) * eb,
                                cudaMemcpyDeviceToDevice, g->stream),
             "loopback copy");
      }
      ck(g, cudaStreamSynchronize(g->stream), "sync");
      lb_barrier(g, lb);                                        // senders may reuse buffers
    }
    return;
  }
  if (!x->comm) fail(g, SG_ENCCL, "communicator was aborted");
  // both arrays in one NCCL group: one collective launch per exchange
  nck(g, x->nccl->groupStart(), "ncclGroupStart");
  for (int p = 0; p < R; ++p) {
    const int64_t sc = soff[p + 1] - soff[p], rc = roff[p + 1] - roff[p];
    for (int pass = 0; pass < 2; ++pass) {
      const void *send = pass ? send2 : send1;
      void *recv = pass ? recv2 : recv1;
      const size_t eb = pass ? eb2 : eb1;
      if (!send) continue;
      if (sc > 0)
        nck(g, x->nccl->send((const char *)send + soff[p] * eb, (size_t)sc * eb, ncclUint8, p, x->comm,
                             g->stream), "ncclSend");
      if (rc > 0)
        nck(g, x->nccl->recv((char *)recv + roff[p] * eb, (size_t)rc * eb, ncclUint8, p, x->comm,
                             g->stream), "ncclRecv");
    }
  }
  nck(g, x->nccl->groupEnd(), "ncclGroupEnd");
  nccl_wait(g, "ncclSend/ncclRecv");
}

void x_alltoallv(sg_graph *g, const void *send, const int64_t *soff, void *recv,
                 const int64_t *roff, size_t eb) {
  x_alltoallv2(g, send, recv, eb, nullptr, nullptr, 0, soff, roff);
}

void x_barrier(sg_graph *g) {
  Exchange *x = g->xch;
  if (x->lb) {
    lb_barrier(g, x->lb);
    return;
  }
  int64_t one = 1;
  std::vector<int64_t> all((size_t)x->world);
  x_allgather_i64(g, &one, 1, all.data());     // returns after every rank contributed
}

void x_share_buffers(sg_graph *g, void *const *mine, int nbuf, std::vector<void *> &all,
                     std::vector<void *> &opened) {
  Exchange *x = g->xch;
  const int R = x->world, me = x->rank;
  all.assign((size_t)R * nbuf, nullptr);
  opened.clear();
  if (x->lb) {
    std::vector<int64_t> v((size_t)nbuf), a((size_t)R * nbuf);
    for (int i = 0; i < nbuf; ++i) v[(size_t)i] = (int64_t)(intptr_t)mine[i];
    x_allgather_i64(g, v.data(), nbuf, a.data());
    for (size_t i = 0; i < a.size(); ++i) all[i] = (void *)(intptr_t)a[i];
    return;
  }
  // NCCL backend: one process per GPU; IPC handles travel as int64 words
  static_assert(sizeof(cudaIpcMemHandle_t) % 8 == 0, "IPC handle size");
  const int W = (int)(sizeof(cudaIpcMemHandle_t) / 8);
  std::vector<int64_t> v((size_t)nbuf * W), a((size_t)R * nbuf * W);
  for (int i = 0; i < nbuf; ++i) {
    cudaIpcMemHandle_t h;
    memset(&h, 0, sizeof h);
    if (mine[i]) ck(g, cudaIpcGetMemHandle(&h, mine[i]), "cudaIpcGetMemHandle");
    memcpy(v.data() + (size_t)i * W, &h, sizeof h);
  }
  x_allgather_i64(g, v.data(), (int64_t)nbuf * W, a.data());
  for (int r = 0; r < R; ++r)
    for (int i = 0; i < nbuf; ++i) {
      if (r == me) {
        all[(size_t)r * nbuf + i] = mine[i];
        continue;
      }
      cudaIpcMemHandle_t h;
      memcpy(&h, a.data() + ((size_t)r * nbuf + i) * W, sizeof h);
      void *p = nullptr;
      ck(g, cudaIpcOpenMemHandle(&p, h, cudaIpcMemLazyEnablePeerAccess), "cudaIpcOpenMemHandle");
      all[(size_t)r * nbuf + i] = p;
      opened.push_back(p);
    }
}

void x_release_buffers(sg_graph *g, std::vector<void *> &opened) {
  x_barrier(g);
  for (void *p : opened) cudaIpcCloseMemHandle(p);
  opened.clear();
}

}  // namespace sg

// ---------------------------------------------------------------- C ABI
extern "C" sg_status sg_loopback_create(int32_t world, sg_loopback **out) {
  if (!out || world < 1) return SG_EINVAL;
  sg_loopback *lb = new sg_loopback();
  lb->world = world;
  lb->hv.resize((size_t)world);
  lb->dptr.resize((size_t)world);
  lb->doff.resize((size_t)world);
  *out = lb;
  return SG_OK;
}

extern "C" void sg_loopback_destroy(sg_loopback *lb) { delete lb; }

extern "C" sg_status sg_nccl_unique_id(uint8_t *out128) {
  if (!out128) return SG_EINVAL;
  std::string why;
  sg::NcclApi *api = sg::nccl_api(&why);
  if (!api) return SG_ENCCL;
  ncclUniqueId uid;
  if (api->getUniqueId(&uid) != ncclSuccess) return SG_ENCCL;
  static_assert(sizeof(uid) == 128, "ncclUniqueId is 128 bytes");
  memcpy(out128, &uid, sizeof(uid));
  return SG_OK;
}
