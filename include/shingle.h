/*
 * shingle.h — C ABI of libshingle.so, the B200 (sm_100a) implementation of the
 * data-parallel hot path of Wu & Kalyanaraman's GPU Shingling (gpClust,
 * IPDPSW 2013): the two-pass min-wise shingle generation of Gibson et al.
 *
 * Citations "P:Lx-y" are lines of the paper text (reference PAPER.md);
 * "AMB-n" are the readings of silent/garbled passages fixed in DESIGN.md §3.
 *
 * Conventions for every call:
 *  - plain C types only; no exceptions cross the ABI; every call returns an
 *    sg_status (or void for destroy);
 *  - host pointers are borrowed for the duration of the call only; device
 *    memory is owned by the handle and released by shingle_graph_destroy;
 *  - all device work is enqueued on the handle's stream (sg_dist.stream, or a
 *    stream the library creates); each call returns when its stage has
 *    completed on the device (it synchronises the stream);
 *  - after SG_ECUDA or SG_ENCCL the handle is poisoned: every later call
 *    except destroy / sg_last_error returns the same status;
 *  - the library never falls back to a CPU implementation: without a usable
 *    CUDA device shingle_graph_create returns SG_ECUDA.
 */
#ifndef SHINGLE_H
#define SHINGLE_H

#include <stdint.h>

#if defined(__GNUC__)
#define SG_API __attribute__((visibility("default")))
#else
#define SG_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

typedef enum sg_status {
    SG_OK = 0,
    SG_EINVAL = 1,     /* invalid argument or invalid CSR (see create) */
    SG_ENOMEM = 2,     /* device allocation failed (sg_last_error names the bytes) */
    SG_ESTATE = 3,     /* call out of order (see the state machine below) */
    SG_ECUDA = 4,      /* CUDA error / no device; the handle is poisoned */
    SG_ENCCL = 5,      /* NCCL error in a multi-GPU exchange; handle poisoned */
    SG_EOVERFLOW = 6   /* a count exceeds 2^32 - 1 (members / rows are u32) */
} sg_status;

typedef struct sg_graph sg_graph;

/* create() flags */
#define SG_DEVICE_PTRS 0x1u   /* row_ptr / col are device pointers (on dist->device) */
#define SG_NO_VALIDATE 0x2u   /* skip the CSR validation (caller guarantees it)   */
#define SG_HOST_CSR    0x4u   /* out-of-core entries: col stays in host memory, page-locked */
                              /* and mapped (cudaHostRegister), and the kernels read it over */
                              /* the host link; only row_ptr is copied to HBM.  The caller  */
                              /* keeps `col` alive and unchanged until the handle is         */
                              /* destroyed or re-loaded.                   */
#define SG_REPORT_HOST 0x10   /* report_dense_subgraphs mode flag: host union-find */

/* Multi-GPU description: one process (or, with loopback, one host thread) per
 * rank, vertex-range sharding, owner-routed exchange before each grouping
 * (DESIGN.md §7).  NULL = one GPU, current device, library-created stream. */
typedef struct sg_dist {
    int32_t rank;              /* 0 <= rank < world */
    int32_t world;             /* number of ranks (>= 1) */
    int32_t device;            /* CUDA device ordinal used by this rank */
    void *stream;              /* cudaStream_t to enqueue on, or NULL */
    const uint8_t *nccl_uid;   /* 128-byte ncclUniqueId (world > 1, NCCL backend) */
    void *loopback;            /* sg_loopback* (world > 1, in-process test backend) or NULL */
    uint32_t flags;            /* SG_DIST_EXCHANGE: run the owner-routed exchange path even */
                               /* at world == 1 (a one-rank NCCL communicator or loopback   */
                               /* group; exercises the multi-GPU transport on one GPU)      */
                               /* SG_DIST_PEER: fused exchange (below)                      */
} sg_dist;

#define SG_DIST_EXCHANGE 0x1u
/* SG_DIST_PEER — fused partition + transfer over peer memory (SURVEY §8(f)
 * N2): every rank exposes one receive buffer per level to all
 * ranks (NCCL backend: CUDA IPC handles exchanged over the communicator, the
 * peers' buffers mapped into this process — NVLink / NVSwitch P2P; loopback:
 * the device pointers of the other virtual ranks), and the owner-partition
 * kernel stores each <shingle, generator> pair straight into its owner's
 * receive buffer at its final position, so no send buffer is written and no
 * NCCL send / recv runs.  The received layout, and hence every output, is
 * identical to the send / recv path.  Ranks synchronise with a barrier
 * before a chunk is written (the owners finished grouping the previous one)
 * and after (all pairs delivered).  Needs P2P access between the ranks'
 * devices (NCCL backend) — SG_ECUDA otherwise. */
#define SG_DIST_PEER 0x2u

/* ------------------------------------------------------------------------ */
/* shingle_graph_create — ingest an unweighted G(V, E) given as adjacency   */
/* lists ("the graph is made available as an adjacency list";   */
/* one contiguous array + boundary marks = CSR).                */
/*   n        number of vertices; 0 <= n < P = 2^31 - 1 (AMB-1: ids must be */
/*            < P for (A*v + B) % P to be a bijection)          */
/*   nnz      number of adjacency entries (2m for an undirected graph)      */
/*   row_ptr  int64[n+1], row_ptr[0] = 0, row_ptr[n] = nnz, non-decreasing  */
/*   col      int32[nnz], each row strictly increasing, 0 <= col < n         */
/*            (AMB-8: duplicates rejected; self-loops/asymmetry accepted)   */
/*   flags    SG_DEVICE_PTRS, SG_NO_VALIDATE                                */
/*   dist     NULL or the rank description above                           */
/*   out      receives the handle (NULL on failure)                         */
/* The whole CSR is global; each rank copies its own row range into HBM.   */
/* Errors: SG_EINVAL (bad arguments / CSR), SG_ENOMEM, SG_ECUDA, SG_ENCCL.  */
/* ------------------------------------------------------------------------ */
SG_API sg_status shingle_graph_create(int64_t n, int64_t nnz, const int64_t *row_ptr,
                               const int32_t *col, uint32_t flags, const sg_dist *dist,
                               sg_graph **out);

/* ------------------------------------------------------------------------ */
/* shingle_graph_load — replace the resident graph of an existing handle by  */
/* a new CSR (same arguments and validation as create), keeping the handle's */
/* device, stream, private memory pool and communicator: the ingest step of  */
/* a long-lived handle that shingles one graph after another (serving).     */
/* Frees both passes' outputs; state -> created.  world > 1: collective.    */
/* Errors: as create.  After a failed load no graph is resident and pass     */
/* returns SG_ESTATE until a load succeeds.                                  */
SG_API sg_status shingle_graph_load(sg_graph *g, int64_t n, int64_t nnz, const int64_t *row_ptr,
                                    const int32_t *col, uint32_t flags);

/* ------------------------------------------------------------------------ */
/* shingle_pass — one shingling pass (Alg. 1).      */
/* First call: Pass I over G.  Second call (after group_by_shingle): Pass II */
/* over G_I, whose rows are the member lists L(s) of the first-level         */
/* shingles with |L| >= s (S1', AMB-6).                          */
/* For every row with at least s entries and every trial       */
/* j < c: the s smallest h_j(v) = (A_j v + B_j) mod P over the row (AMB-7),  */
/* folded into a within-trial shingle id (AMB-4: s=1: h1; s=2:               */
/* h1*2^31 + h2; s>=3: 64-bit splitmix fold).  (A_j, B_j) come from a        */
/* splitmix64 stream seeded with `seed` (AMB-2).                            */
/*   s in [1, 8] (s "typically under 10"), c in [1, 1024].       */
/* Errors: SG_EINVAL (s, c), SG_ESTATE (wrong order), SG_ENOMEM, SG_ECUDA,  */
/* SG_EOVERFLOW (rows * c >= 2^32 on one rank).                              */
/* ------------------------------------------------------------------------ */
SG_API sg_status shingle_pass(sg_graph *g, int32_t s, int32_t c, uint64_t seed);

/* ------------------------------------------------------------------------ */
/* group_by_shingle — "a sorting is done to gather all vertices that         */
/* generated each shingle ... once for each random trial" (P:L404-410,       */
/* AMB-5): per trial, the <shingle, generator> pairs of the last pass are    */
/* grouped into tuples <s_j, L(s_j)>, giving G_I after pass I   */
/* and G_II after pass II.  Canonical order (AMB-19): trials    */
/* ascending; within a trial, groups by key = splitmix64-finaliser(id)       */
/* ascending; members ascending.  With world > 1 the pairs are first routed */
/* to the rank owning their key (NCCL all-to-all).                           */
/* Errors: SG_ESTATE, SG_ENOMEM, SG_ECUDA, SG_ENCCL, SG_EOVERFLOW.           */
/* ------------------------------------------------------------------------ */
SG_API sg_status group_by_shingle(sg_graph *g);

/* ------------------------------------------------------------------------ */
/* report_dense_subgraphs — Phase III, approach 2: */
/* union-find of size n; for each connected component of G_II, union the    */
/* vertices of G that constitute its first- and second-level shingles       */
/* (mode 0, AMB-9) or that generated its first-level shingles (mode 1).     */
/*   labels     host int32[n], caller-allocated; labels[v] = smallest vertex */
/*              of v's cluster (AMB-10); clusters smaller than min_size are  */
/*              reported as singletons (labels[v] = v).                      */
/*   n_clusters receives the number of clusters with >= max(2, min_size)     */
/*              vertices (may be NULL).                                      */
/*   mode       0 or 1, optionally | SG_REPORT_HOST.  Default: on the device */
/*              (lock-free union-find over n, one thread per S1' node and per  */
/*              G_II pair, stage "report" of sg_get_stage_ms); with the flag:  */
/*              the same union-find on the host (G_I, G_II copied back).       */
/* Outside the timed two-pass hot path.  Requires state GROUPED2 and         */
/* world == 1 (SG_EINVAL otherwise: gather G_II with sg_get_groups).         */
/* ------------------------------------------------------------------------ */
SG_API sg_status report_dense_subgraphs(sg_graph *g, int32_t mode, int32_t min_size, int32_t *labels,
                                 int64_t *n_clusters);

/* ------------------------------------------------------------------------ */
/* report_overlapping_clusters — Phase III, approach 1:        */
/* "enumerate all connected components in G_II ... for each connected      */
/* component, report the set of all vertices in G that constitute the       */
/* first-level shingles of that component as a cluster" (clusters may       */
/* overlap).  Components join S1' nodes through shared G_II groups.         */
/*   mode     0: constituents (top-s1 vertices of the smallest generator's  */
/*            row under H1[j], AMB-9/AMB-18); 1: the generators L(s).       */
/*   min_size clusters with fewer vertices are not reported.                */
/*   offs     host int64[C+1], verts host uint32[V]: cluster i is            */
/*            verts[offs[i], offs[i+1]), vertices ascending; clusters in     */
/*            order of their smallest S1' index.  Caller-allocated; caps =   */
/*            {C+1, V}.  Both NULL: only counts <- {C, V} (two-call pattern; */
/*            the sizing call's result is kept on the host for the next     */
/*            filling call with the same mode and min_size, then released). */
/* Union-find over S1', constituent emission, radix sort + unique on the    */
/* device; the host splits the sorted list.  Untimed; state GROUPED2,       */
/* world == 1.  Errors: SG_EINVAL (mode, NULL counts, caps too small,       */
/* world > 1),                                                               */
/* SG_ESTATE, SG_ENOMEM, SG_ECUDA, SG_EOVERFLOW (> 2^31 constituents).      */
/* ------------------------------------------------------------------------ */
SG_API sg_status report_overlapping_clusters(sg_graph *g, int32_t mode, int32_t min_size,
                                             int64_t *offs, uint32_t *verts, const int64_t caps[2],
                                             int64_t counts[2]);

/* ------------------------------------------------------------------------ */
/* sg_cluster_density — Eq. 6: density of a cluster =       */
/* #(edges in the cluster) / #(possible edges) = e / C(k, 2), averaged over */
/* the clusters of a partition (the paper: 0.75 +- 0.28 for gpClust on the  */
/* 2M GOS graph, Table IV context).                                          */
/*   labels   host int32[n], labels[v] in [0, n) names v's cluster (e.g. the */
/*            output of report_dense_subgraphs); borrowed, copied to HBM.    */
/*   min_size clusters with fewer than max(2, min_size) vertices are skipped.*/
/*   mean, stddev (population) and n_clusters receive the statistics over    */
/*   the counted clusters (0 when none); each may be NULL.                   */
/* Intra-cluster edges are counted on the device (one warp per row, over   */
/* the resident CSR; undirected edges are stored twice, AMB-11).  Any state */
/* after create; world == 1.  Errors: SG_EINVAL (NULL labels, label out of  */
/* range, world > 1), SG_ENOMEM, SG_ECUDA.                                  */
/* ------------------------------------------------------------------------ */
SG_API sg_status sg_cluster_density(sg_graph *g, const int32_t *labels, int32_t min_size,
                                    double *mean, double *stddev, int64_t *n_clusters);

/* ------------------------------------------------------------------------ */
/* sg_partition_agreement — the pair counts behind Eq. 2-5 (P:L1038-1060,  */
/* AMB-15): over all unordered vertex pairs (i, j) of G,                    */
/*   TP: same cluster in test and in benchmark;  FP: same in test only;     */
/*   FN: same in benchmark only;                 TN: apart in both.         */
/* PPV = TP/(TP+FP), NPV = TN/(TN+FN), SP = TN/(TN+FP), SE = TP/(TP+FN).    */
/*   test_labels, bench_labels  host int32[n], values in [0, n) (borrowed). */
/*   counts     receives {TP, FP, FN, TN} (exact 64-bit integers).          */
/* Marginal histograms and a radix sort + run-length encode of the joint    */
/* (test, benchmark) cells on the device.  Any state after create; world   */
/* == 1.  Errors: SG_EINVAL (NULL, label out of range, world > 1),         */
/* SG_EOVERFLOW, SG_ENOMEM, SG_ECUDA.                                      */
/* ------------------------------------------------------------------------ */
SG_API sg_status sg_partition_agreement(sg_graph *g, const int32_t *test_labels,
                                        const int32_t *bench_labels, int64_t counts[4]);

/* ------------------------------------------------------------------------ */
/* sg_connected_components — the connected components of G, the            */
/* decomposition pClust applies before shingling: no dense     */
/* subgraph spans two components, so each can be shingled on its own.     */
/*   labels        host int32[n], caller-allocated; labels[v] = smallest    */
/*                 vertex of v's component (isolated vertices: v).          */
/*   n_components  receives the number of components (may be NULL).        */
/* Lock-free union-find over n on the device (one warp per CSR row, each    */
/* stored entry (u, v) is an undirected edge).  Any state after create;   */
/* world == 1.                                                              */
/* Errors: SG_EINVAL (NULL labels, world > 1), SG_ENOMEM, SG_ECUDA.       */
/* ------------------------------------------------------------------------ */
SG_API sg_status sg_connected_components(sg_graph *g, int32_t *labels, int64_t *n_components);

/* Return the handle to state CREATED (CSR kept, results dropped) so the two */
/* passes can be run again, e.g. by a benchmark.                             */
SG_API sg_status shingle_graph_reset(sg_graph *g);

SG_API void shingle_graph_destroy(sg_graph *g);

/* Last error message of the handle (or of the calling thread if g == NULL). */
SG_API const char *sg_last_error(const sg_graph *g);

/* ------------------------------------------------------------------------ */
/* Getters (host buffers; two-call pattern: NULL buffers report sizes).      */
/* ------------------------------------------------------------------------ */

/* counts[0..15] = n, this rank's first row, rows on this rank, n_e (pass-I  */
/* rows, global), |S1| (G_I groups), |S1'| (pass-II rows), |S2| (G_II        */
/* groups), P1 pairs, P2 pairs, state, E2 (pass-II entries = sum of |L| over */
/* S1'), device-kernel launches since create / the last reset, trial chunks  */
/* of pass I and of pass II (negative: keys computed inside the grouping,    */
/* DESIGN.md §6.3), world (ranks of the exchange), 1 if the owner-routed   */
/* exchange path is on (world > 1 or SG_DIST_EXCHANGE) else 0.  Global      */
/* counts are summed over ranks.  The                                        */
/* environment variable SG_MEM_BUDGET (bytes, read at create) caps the HBM   */
/* the planner assumes, to exercise the chunked paths on small graphs.      */
/* world > 1: collective (every rank calls it; it sums the counts once per   */
/* level), like shingle_pass and group_by_shingle.  Other getters are local. */
SG_API sg_status sg_get_counts(const sg_graph *g, int64_t counts[16]);

/* Shingle matrix of pass `level` (1 or 2) on this rank: ids[rows x c]      */
/* row-major (rows ascending: pass I = vertices with deg >= s1 ascending;   */
/* pass II = S1' indices ascending), plus the row's generator value in       */
/* rowid[rows] (pass I: vertex id; pass II: S1' index).                      */
SG_API sg_status sg_get_shingles(sg_graph *g, int32_t level, uint64_t *ids, uint32_t *rowid,
                          int64_t cap_rows, int64_t *rows, int32_t *c);

/* Groups of level 1 (G_I) or 2 (G_II) owned by this rank, canonical order:  */
/*   trial_goffs[c+1] group ranges per trial, ids[G], offs[G+1] (into        */
/*   members), members[Pairs].  caps = {G, Pairs}; counts <- {G, Pairs, c}.  */
SG_API sg_status sg_get_groups(sg_graph *g, int32_t level, int64_t *trial_goffs, uint64_t *ids,
                        int64_t *offs, uint32_t *members, const int64_t caps[2],
                        int64_t counts[3]);

/* The same for the trials [t0, t1) only (grouping is per trial, */
/* AMB-5, so a trial range is a self-contained slice of the level; t1 = -1   */
/* means c).  trial_goffs[t1-t0+1] and offs[G+1] are relative to the first  */
/* group / pair of trial t0; counts <- {G, Pairs, t1 - t0}.  Lets a caller    */
/* read G_II of a 2M- or 640M-edge graph trial by trial (tens of GB in all). */
/* SG_EINVAL unless 0 <= t0 <= t1 <= c.                                      */
SG_API sg_status sg_get_groups_range(sg_graph *g, int32_t level, int32_t t0, int32_t t1,
                                     int64_t *trial_goffs, uint64_t *ids, int64_t *offs,
                                     uint32_t *members, const int64_t caps[2], int64_t counts[3]);

/* Shingle matrix columns [t0, t1) of pass `level`: ids[rows x (t1-t0)]      */
/* row-major (t1 = -1 means c); rowid as in sg_get_shingles.                 */
SG_API sg_status sg_get_shingles_range(sg_graph *g, int32_t level, int32_t t0, int32_t t1,
                                       uint64_t *ids, uint32_t *rowid, int64_t cap_rows,
                                       int64_t *rows, int32_t *c);

/* The S1' map: s1p_group[k] = index (in this rank's G_I, canonical order)   */
/* of first-level shingle k; first global index of this rank in *k0.        */
SG_API sg_status sg_get_s1p(sg_graph *g, int64_t *s1p_group, int64_t cap, int64_t *count, int64_t *k0);

/* Hash pairs of pass `level`: A[c], B[c]. */
SG_API sg_status sg_get_hash_params(sg_graph *g, int32_t level, uint32_t *A, uint32_t *B, int32_t cap);

/* Device milliseconds of the last stages (CUDA events on the handle's      */
/* stream): [0] pass I, [1] group I, [2] pass II, [3] group II, then         */
/* sub-stages [4..18]: select1, hash1, select2, hash2, hist1, scatter1,      */
/* local1, hist2, scatter2, local2, exchange1, exchange2, fine1, fine2,      */
/* report.  At most 19 values; *n receives the number written.*/
SG_API sg_status sg_get_stage_ms(const sg_graph *g, float *ms, int32_t cap, int32_t *n);

/* Multi-GPU in-process test backend: `world` virtual ranks on one device,   */
/* each driven by its own host thread, exchanging through device memcpy.     */
typedef struct sg_loopback sg_loopback;
SG_API sg_status sg_loopback_create(int32_t world, sg_loopback **out);
SG_API void sg_loopback_destroy(sg_loopback *lb);

/* NCCL backend: rank 0 creates the 128-byte ncclUniqueId that every rank    */
/* passes in sg_dist.nccl_uid (broadcast it, e.g. with torch.distributed).   */
/* SG_ENCCL if libnccl.so.2 cannot be loaded.                                */
SG_API sg_status sg_nccl_unique_id(uint8_t *out128);

/* Canonical pass-II dense index: given the all-gathered      */
/* counts all[r * c1 + j] of S1' rows of pass-I trial j on rank r, the local */
/* rows of trial j on `rank` are [first[j], first[j+1]) and row i of trial j */
/* gets k = i + off[j].  first[c1 + 1], off[c1]; returns |S1'| in *total.     */
/* Pure host code (testable without GPU).                                    */
SG_API sg_status sg_s1p_offsets(int32_t world, int32_t rank, int32_t c1, const int64_t *all,
                                int64_t *first, int64_t *off, int64_t *total);

/* Host-side vertex-range partition used by create: splits   */
/* [0, n) into `world` contiguous ranges balancing sum(deg + kappa).  bounds */
/* receives world + 1 row indices.  Pure host code (testable without GPU).   */
SG_API sg_status sg_partition_rows(int64_t n, const int64_t *row_ptr, int32_t world, int64_t kappa,
                            int64_t *bounds);

/* ------------------------------------------------------------------------ */
/* Component sharding: pClust breaks the input graph into  */
/* connected components before shingling.  Shingling only looks */
/* at neighbourhoods, so no shingle, group or dense subgraph spans two       */
/* components: whole components can be shingled on different GPUs with no    */
/* exchange, every vertex taking its label from its own shard (the oracle's  */
/* CC-locality self-check).  Pure host code (no GPU).                        */
/*                                                                           */
/* sg_component_shards: shard[n] <- the shard (0..world-1) of every vertex;  */
/*   components (every stored entry an undirected edge) are placed heaviest  */
/*   first on the least-loaded shard by sum(deg + kappa); load[world]        */
/*   (optional) <- each shard's weight.  SG_EINVAL on a bad CSR.             */
SG_API sg_status sg_component_shards(int64_t n, const int64_t *row_ptr, const int32_t *col,
                                     int32_t world, int64_t kappa, int32_t *shard, int64_t *load);
/* sg_shard_csr: the CSR of shard r over all n vertex ids (rows of the other */
/*   shards empty): row_ptr_out[n+1], col_out[*nnz_out]; NULL outputs ->     */
/*   only *nnz_out (two-call pattern).  Pass it to shingle_graph_create /    */
/*   shingle_graph_load of the shard's GPU (world 1, no exchange).           */
SG_API sg_status sg_shard_csr(int64_t n, const int64_t *row_ptr, const int32_t *col,
                              const int32_t *shard, int32_t r, int64_t *row_ptr_out,
                              int32_t *col_out, int64_t *nnz_out);
/* sg_merge_shard_labels: out[v] = labels[shard[v] * n + v] (labels: the     */
/*   world shards' report_dense_subgraphs labels stacked row by row).        */
SG_API sg_status sg_merge_shard_labels(int64_t n, const int32_t *shard, int32_t world,
                                       const int32_t *labels, int32_t *out);

/* Library version / build string (sm_100a). */
SG_API const char *sg_version(void);

#ifdef __cplusplus
}
#endif

#endif /* SHINGLE_H */
