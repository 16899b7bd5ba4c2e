// kernels.h — host launchers of the libshingle device kernels.
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <atomic>

namespace sg {

// Number of device-kernel launches issued by this library (process-wide).
extern std::atomic<long long> g_launches;

// ---- row selection (kernels_pass.cu) ---------------------------------------
// Pass I rows: local CSR rows with deg >= s.  Two launches with a
// host read of the count in between (the count sizes the next allocations).
// `blk` is device scratch of sel_scratch_elems(nrows_local) int64.
int64_t sel_scratch_elems(int64_t items);
cudaError_t select_csr_count(const int64_t *row_ptr, int64_t nrows_local, int s, int64_t *blk,
                             int64_t *d_total, cudaStream_t st);
cudaError_t select_csr_write(const int64_t *row_ptr, int64_t nrows_local, int s, int64_t row_lo,
                             const int64_t *blk, int64_t *rstart, int32_t *rlen, uint32_t *rowid,
                             cudaStream_t st);
// Pass II rows: groups of G_I (head bits over npairs members) with |L| >= s
// (S1'), in canonical order.
cudaError_t select_groups_count(const uint32_t *head, int64_t npairs, int s, int64_t *blk,
                                int64_t *d_total, cudaStream_t st);
cudaError_t select_groups_write(const uint32_t *head, int64_t npairs, int s, const int64_t *blk,
                                int64_t *rstart, int32_t *rlen, cudaStream_t st);

// ---- min-hash top-s (kernels_pass.cu) --------------------------------------
struct MinhashArgs {
  const int64_t *rstart;
  const int32_t *rlen;
  const uint32_t *entries;
  int64_t nrows;
  const uint32_t *A;              // [c] hash pairs of the whole pass
  const uint32_t *B;
  int32_t t0;                     // first trial of this launch
  int32_t nt;                     // trials in this launch
  int32_t s;
  uint64_t seed;
  uint64_t *keys;                 // [nt][key_stride], key_stride % 8 == 0
  int64_t key_stride;
  unsigned long long *counter;    // zeroed device counter (row tiles)
  unsigned long long *hub_counter;  // zeroed device counter (hub-row blocks)
  int32_t tile_rows = 8;          // rows per warp tile: 8 (long rows) or 16 (short rows)
  uint8_t *kbin = nullptr;        // [nt][key_stride] top key byte (the grouping's coarse bin,
                                  // read by hist_kernel instead of the 8-B keys) or nullptr
};
constexpr int kRowTile = 16;      // key_stride granule (multiple of every tile size)
inline int64_t key_stride_for(int64_t nrows) { return (nrows + kRowTile - 1) / kRowTile * kRowTile; }
cudaError_t minhash(const MinhashArgs &a, int num_sms, cudaStream_t st);
// Rows of <= short_row_max() entries, one row per lane (pass II, DESIGN.md
// §6.1): keys[j][r] for the a.nrows rows of (a.rstart, a.rlen).
cudaError_t minhash_short_rows(const MinhashArgs &a, int num_sms, cudaStream_t st);
int32_t short_row_max();
// Length-class layout of rows: call with h_start == nullptr to count rows per
// class (d_cnt[short_row_max() + 2] = rows of length 0..max, then longer),
// then with the host class starts to write perm / rstart_p / rlen_p (classes
// contiguous, ascending length, longer rows last; order inside a class free).
cudaError_t row_classes(const int64_t *rstart, const int32_t *rlen, int64_t n, unsigned long long *d_cnt,
                        unsigned long long *d_cursor, const unsigned long long *h_start, uint32_t *perm,
                        int64_t *rstart_p, int32_t *rlen_p, cudaStream_t st);

// Recompute shingle ids for (row, trial) requests (getters / report only).
cudaError_t shingle_ids(const int64_t *rstart, const int32_t *rlen, const uint32_t *entries,
                        const uint32_t *A, const uint32_t *B, int32_t s, uint64_t seed,
                        const int64_t *req_row, const int32_t *req_trial, int64_t nreq,
                        uint64_t *ids, cudaStream_t st);

// ---- grouping (kernels_group.cu) -------------------------------------------
struct GroupPlan {
  int32_t c = 0;
  int32_t bits = 0;          // B: final buckets per trial = 2^B (top B key bits)
  int32_t bits1 = 0;         // coarse (first scatter) bits; == bits when single-level
  int64_t nbins = 1;         // 2^bits
  int64_t nb1 = 1;           // 2^bits1
  int64_t nchunks = 0;
  int64_t npairs = 0;
  // device tables (built on the device from the piece table)
  int64_t *chunk_i0 = nullptr;     // [nchunks] row index of the chunk's first pair (implicit values)
  int32_t *chunk_len = nullptr;    // [nchunks]
  int32_t *chunk_trial = nullptr;  // [nchunks]
  int64_t *chunk_in0 = nullptr;    // [nchunks] key / explicit-value index of the chunk's first pair
  int64_t *seg = nullptr;          // [c+1] output position of pair 0 of trial j (global)
  int32_t *trial_chunk0 = nullptr; // [c+1] first chunk of each trial
  int64_t chunk = 4096;            // pairs per chunk (the tables above)
  int32_t local_cap = 0;           // grouping v3: largest coarse bucket sorted by a CTA (0: default)
  int32_t fine_bits = 0;           // grouping v3: fine (counting-sort) bits after the coarse bits
};

struct GroupArgs {
  GroupPlan plan;
  const uint64_t *keys;        // [npairs] pre-group keys (per-trial segments)
  const uint8_t *kbin = nullptr;   // top byte of each key, same indexing (or nullptr)
  const uint32_t *vals;        // explicit generator values, or nullptr:
  const uint32_t *rowid;       //   val = rowid[i - seg[j]] if rowid, else
  uint32_t val_base;           //   val = val_base + (i - seg[j])
  // scratch (device)
  uint32_t *counts;            // [nchunks][nb1]
  uint32_t *bstart1;           // [c][nb1] coarse bucket start within the trial segment
  uint32_t *bsize1;            // [c][nb1]
  uint32_t *bstart;            // [c][nbins] final bucket start (== bstart1 if single-level)
  uint32_t *bsize;             // [c][nbins]
  uint64_t *akeys;             // [npairs] coarse-bucketed pairs
  uint32_t *avals;
  uint8_t *fbin = nullptr;     // [npairs] fine digit (key bits 48..55) of the coarse-bucketed
                               // pairs, 16-bit two-level plans only (or nullptr)
  // fused exchange (SG_DIST_PEER): owner partition writes bin d's pairs into
  // rank d's receive buffers (device arrays of nb1 peer pointers) instead of
  // akeys / avals
  uint64_t *const *peer_keys = nullptr;
  uint32_t *const *peer_vals = nullptr;
  uint64_t *bkeys;             // [npairs] final-bucketed pairs (== akeys if single-level)
  uint32_t *bvals;
  uint32_t *big_list;          // [c*nbins] bucket ids with size > 4096 (global sort)
  uint32_t *big_count;         // [1] (zeroed by the caller)
  uint32_t *mid_list;          // [c*nbins] bucket ids with 1024 < size <= 4096 (CTA sort)
  uint32_t *mid_count;         // [1] (zeroed by the caller)
  uint32_t *gcur = nullptr;    // v3: [c][nb1] running bucket reservation cursors
  unsigned long long *seg_count = nullptr;   // v3: one-key fine buckets of > 8 members left
  int64_t *seg_pos = nullptr;                //   unsorted in `members`: output position,
  uint32_t *seg_len = nullptr;               //   length (capacity npairs / 9 + 1)
  // outputs
  uint32_t *members;           // [npairs]
  uint32_t *head;              // [(npairs+31)/32], zeroed by the launcher
  uint64_t *okeys = nullptr;   // [npairs] sorted keys (optional; multi-rank getters)
};

// ---- multi-rank helpers (kernels_pass.cu) ----------------------------------
// counts[j] = number of rows whose rstart lies in [seg[j], seg[j+1]) (zeroed by caller)
cudaError_t rows_per_trial(const int64_t *rstart, int64_t nrows, const int64_t *seg, int32_t c,
                           unsigned long long *counts, cudaStream_t st);
// rowid[i] = i + off[j] for the trial j with first[j] <= i < first[j+1]
cudaError_t assign_rowid(uint32_t *rowid, int64_t nrows, const int64_t *first, const int64_t *off,
                         int32_t c, cudaStream_t st);

int64_t group_local_capacity();
int split_mode(bool fine);        // ranking mode of the split kernels (SG_SPLIT_FINE / _COARSE)
int split_atomic();              // a split may deliver pairs out of generator order
int64_t group_chunk_pairs();     // pairs per partition chunk (hist and scatter)
int32_t group_max_fanout();      // bins of one split pass (owner ranks <= this)
// Bucket plan for trial segments of at most `maxseg` pairs.
void group_bits(int64_t maxseg, int32_t *bits, int32_t *bits1);
// Fill plan.chunk_* (plan.nchunks entries) from the piece table (device
// pointers; pieces ordered by trial, chunks of group_chunk_pairs() pairs).
cudaError_t group_chunk_tables(const GroupPlan &plan, const int32_t *p_trial, const int64_t *p_in0,
                               const int64_t *p_len, const int64_t *p_row0,
                               const int64_t *p_chunk0, int32_t npieces, cudaStream_t st);
cudaError_t group_hist(const GroupArgs &g, cudaStream_t st);
cudaError_t group_offsets(const GroupArgs &g, cudaStream_t st);
cudaError_t group_colscan(const GroupArgs &g, cudaStream_t st);   // chunk prefixes + bsize1 only
cudaError_t group_scatter(const GroupArgs &g, int num_sms, cudaStream_t st);
cudaError_t group_scatter2(const GroupArgs &g, cudaStream_t st);   // two-level plans only
// Sort every final bucket and write members + head bits: warp tier, then the
// mid and big tiers over the lists the warp tier filled (no host sync).
cudaError_t group_local(const GroupArgs &g, int num_sms, cudaStream_t st);
// Global-memory sort of the buckets listed in big_list (count on the device).
cudaError_t group_big(const GroupArgs &g, int num_sms, cudaStream_t st);

// ---- grouping v3 (kernels_sort.cu): coarse totals by the
// top plan.bits1 (<= 11) key bits over chunks of group_c_chunk_pairs() pairs
// (plan.chunk), an unordered coarse scatter with per-bucket atomic
// reservations (gcur), then per coarse bucket a counting sort by the next
// plan.fine_bits (<= 14) bits into a per-CTA scratch (bkeys / bvals,
// group_c_scratch_pairs() pairs) and a (key, member) sort of every fine bucket.
int64_t group_c_chunk_pairs();
int32_t group_c_local_cap();
int64_t group_c_scratch_pairs(int num_sms);
void group_c_bits(int64_t maxseg, int32_t *bits1, int32_t *fine_bits);
cudaError_t group_c_hist(const GroupArgs &g, int num_sms, cudaStream_t st);     // + bucket starts
cudaError_t group_c_scatter(const GroupArgs &g, int num_sms, cudaStream_t st);
cudaError_t group_c_bucket(const GroupArgs &g, int num_sms, cudaStream_t st);   // + big
// Sort the members of every listed segment ascending (count read on the device).
cudaError_t group_c_segsort(const GroupArgs &g, int num_sms, cudaStream_t st);
cudaError_t group_binscan(const GroupArgs &g, cudaStream_t st);   // bstart1 = scan of bsize1 per trial

// ---- Phase III on the device (kernels_report.cu) ---------------------------
struct ReportArgs {
  int64_t n = 0;                    // vertices of G
  int32_t mode = 0;                 // 0 constituents, 1 generators (AMB-9)
  int32_t min_size = 1;
  int32_t s1 = 0, s2 = 0;
  const uint32_t *A1 = nullptr, *B1 = nullptr, *A2 = nullptr, *B2 = nullptr;   // device [c]
  const int64_t *row_ptr = nullptr; // CSR of G (device, single rank: rebased = global)
  const uint32_t *col = nullptr;
  const uint32_t *members1 = nullptr;   // G_I members (canonical order)
  int64_t rows1 = 0;                // pass-I rows: trial j owns members1[j*rows1, (j+1)*rows1)
  const int64_t *rstart2 = nullptr; // S1' node k: its group L(k) = members1[rstart2[k], +rlen2[k])
  const int32_t *rlen2 = nullptr;
  int64_t nk = 0;                   // |S1'|
  const uint32_t *members2 = nullptr;   // G_II members (S1' indices)
  const uint32_t *head2 = nullptr;      // G_II head bits
  int64_t npairs2 = 0;
  int64_t rows2 = 0;                // pass-II rows (= nk): trial t owns [t*rows2, (t+1)*rows2)
  // mode 0, s2 <= 2: the S1' nodes in length-class order (row_classes) for
  // the per-node second-level constituents (rows [0, nshort2) of <= 8 entries)
  const uint32_t *perm2 = nullptr;
  const int64_t *rstart2p = nullptr;
  const int32_t *rlen2p = nullptr;
  int64_t nshort2 = 0;
  int32_t c2 = 0;
};
// parent/size: device uint32[n]; rep1: device uint32[nk]; labels: device
// int32[n]; *d_nc receives the cluster count.
cudaError_t report_device(const ReportArgs &a, uint32_t *parent, uint32_t *rep1, uint32_t *size,
                          int32_t *labels, unsigned long long *d_nc, int num_sms, cudaStream_t st);

// Phase III approach 1 (overlapping clusters): parentK uint32[nk]; eoff
// int64[nk] (mode 1); keys / keys_sorted uint64[nkeys] (mode 0: nk * s1, mode
// 1: sum of |L(k)|); afterwards keys[0, *d_nuniq) = sorted unique
// (component root << 32 | vertex), sentinels ~0 last.
size_t overlap_temp_bytes(int64_t nk, int64_t nkeys);
cudaError_t overlap_device(const ReportArgs &a, uint32_t *parentK, int64_t *eoff, uint64_t *keys,
                           uint64_t *keys_sorted, int64_t nkeys, void *temp, size_t temp_bytes,
                           int64_t *d_nuniq, int num_sms, cudaStream_t st);

// Cluster density (Eq. 6): e2[label] = 2 x intra-cluster edges, size[label] =
// vertices, both device [n] and zeroed here; labels device int32[n] in [0, n).
cudaError_t density_device(const int64_t *row_ptr, const uint32_t *col, int64_t n,
                           const int32_t *labels, unsigned long long *e2, uint32_t *size,
                           int num_sms, cudaStream_t st);

// Partition agreement (Eq. 2-5): t, b device int32[n] in [0, n); ct, cb, cj
// uint32[n], key, key2 uint64[n] scratch; d_out3 <- {sum C(n_tb,2),
// sum C(n_t,2), sum C(n_b,2)}.
size_t agreement_temp_bytes(int64_t n);
cudaError_t agreement_device(const int32_t *t, const int32_t *b, int64_t n, uint32_t *ct,
                             uint32_t *cb, uint32_t *cj, uint64_t *key, uint64_t *key2, void *temp,
                             size_t temp_bytes, int64_t *d_runs, unsigned long long *d_out3,
                             int num_sms, cudaStream_t st);

// Connected components of G: parent uint32[n] scratch, labels device int32[n]
// <- smallest vertex of the component.
cudaError_t components_device(const int64_t *row_ptr, const uint32_t *col, int64_t n,
                              uint32_t *parent, int32_t *labels, int num_sms, cudaStream_t st);

// ---- getters (kernels_group.cu) --------------------------------------------
cudaError_t popcount_words(const uint32_t *w, int64_t nwords, unsigned long long *d_out,
                           cudaStream_t st);
cudaError_t sum_i32(const int32_t *a, int64_t n, unsigned long long *d_out, cudaStream_t st);

}  // namespace sg
