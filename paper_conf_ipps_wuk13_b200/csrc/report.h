// report.h — Phase III on the host (untimed): P:L483-488.
#pragma once

#include <stdint.h>

#include <vector>

namespace sg {

struct ReportInput {
  int64_t n = 0;
  int32_t s1 = 0, s2 = 0;
  const uint32_t *A1 = nullptr, *B1 = nullptr, *A2 = nullptr, *B2 = nullptr;
  // first-level shingles in S1' (k = 0..nk-1): trial, id, generator list L(k)
  int64_t nk = 0;
  const int32_t *trial1 = nullptr;
  const uint64_t *id1 = nullptr;
  const int64_t *loff = nullptr;    // [nk+1]
  const uint32_t *lmem = nullptr;   // vertex ids
  // second-level shingles (G_II groups h = 0..nh-1): trial, id, members K(h)
  int64_t nh = 0;
  const int32_t *trial2 = nullptr;
  const uint64_t *id2 = nullptr;
  const int64_t *koff = nullptr;    // [nh+1]
  const uint32_t *kmem = nullptr;   // S1' indices
  // CSR of G (host) for s1 >= 3 constituent recomputation
  const int64_t *row_ptr = nullptr;
  const int32_t *col = nullptr;
};

// mode 0: constituents; mode 1: generators (DESIGN.md AMB-9).  Returns the
// number of clusters with >= max(2, min_size) vertices.
int64_t report_host(const ReportInput &in, int32_t mode, int32_t min_size, int32_t *labels);

// splitmix64 hash-pair stream (AMB-2), host side of the product path.
void hash_pairs(uint64_t seed, int32_t c, uint32_t *A, uint32_t *B);

}  // namespace sg
