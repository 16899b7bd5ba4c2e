// exchange.h — multi-GPU transport of libshingle.
//
// Two backends behind one interface:
//  * NCCL (one process per GPU; libnccl.so.2 is loaded with dlopen so the
//    library also loads on machines without NCCL; the communicator is built
//    from a 128-byte ncclUniqueId broadcast by the caller, e.g. through
//    torch.distributed);
//  * loopback (world virtual ranks inside one process, one host thread per
//    rank, all on one device): collectives are host barriers + device
//    memcpys.  It exercises the whole multi-rank path on a single GPU.
#pragma once

#include <vector>

#include "sg_internal.cuh"

namespace sg {

Exchange *exchange_create(sg_graph *g, const sg_dist *dist);
void exchange_destroy(Exchange *x);
// A rank that fails inside a call marks the loopback group broken so its
// peers leave their barriers with SG_ESTATE instead of waiting forever.
void exchange_abort(Exchange *x);

// all[r * n + i] = value i of rank r (host arrays).
void x_allgather_i64(sg_graph *g, const int64_t *mine, int64_t n, int64_t *all);
int64_t exchange_sum(sg_graph *g, int64_t v);
int64_t exchange_min(sg_graph *g, int64_t v);
// Device all-to-all-v: rank r sends send[soff[d] .. soff[d+1]) (elements of
// eb bytes) to rank d and receives rank s's block into recv[roff[s] ..).
// soff / roff are host arrays of world + 1 element offsets.  Enqueued on the
// handle's stream; returns when the transfer has completed.
void x_alltoallv(sg_graph *g, const void *send, const int64_t *soff, void *recv,
                 const int64_t *roff, size_t eb);

// ---- fused exchange over peer memory (SG_DIST_PEER)
// Barrier over the ranks (host: returns when every rank has called it).
void x_barrier(sg_graph *g);
// Publish `nbuf` device buffers of this rank (allocated with cudaMalloc) and
// map every rank's: all[r * nbuf + i] is rank r's buffer i, usable by this
// rank's kernels (NCCL backend: CUDA IPC handles exchanged over the
// communicator and opened here; loopback: the peers' pointers, same device).
// `opened` receives the mappings this rank must release.
void x_share_buffers(sg_graph *g, void *const *mine, int nbuf, std::vector<void *> &all,
                     std::vector<void *> &opened);
// Barrier (no rank still writes into a peer buffer), then unmap `opened`.
void x_release_buffers(sg_graph *g, std::vector<void *> &opened);
// Two arrays with the same element offsets (keys and generators) in one
// exchange: one NCCL group (send2 == nullptr: one array).
void x_alltoallv2(sg_graph *g, const void *send1, void *recv1, size_t eb1, const void *send2,
                  void *recv2, size_t eb2, const int64_t *soff, const int64_t *roff);

}  // namespace sg
