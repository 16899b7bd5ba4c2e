// shards.cpp — pClust's decomposition (the input graph is broken
// into connected components before shingling) as a sharding option of
// libshingle.  Shingling only looks at neighbourhoods: the
// constituents and the generators of a shingle are neighbours of one vertex,
// so no shingle, group or dense subgraph spans two components (the oracle's
// CC-locality self-check vii).  Whole components can therefore be shingled
// on different GPUs with no exchange at all, each vertex taking its label
// from its own shard.  Host code (plain C++), no device work.
#include <algorithm>
#include <numeric>
#include <queue>
#include <vector>

#include "../../include/shingle.h"

namespace {

int64_t find_root(std::vector<int64_t> &p, int64_t x) {
  while (p[(size_t)x] != x) {
    p[(size_t)x] = p[(size_t)p[(size_t)x]];
    x = p[(size_t)x];
  }
  return x;
}

}  // namespace

extern "C" {

sg_status sg_component_shards(int64_t n, const int64_t *row_ptr, const int32_t *col, int32_t world,
                              int64_t kappa, int32_t *shard, int64_t *load) {
  if (n < 0 || world < 1 || (n > 0 && (!row_ptr || !shard)) || kappa < 0) return SG_EINVAL;
  if (n == 0) {
    if (load)
      for (int32_t r = 0; r < world; ++r) load[r] = 0;
    return SG_OK;
  }
  const int64_t nnz = row_ptr[n];
  if (row_ptr[0] != 0 || nnz < 0 || (nnz > 0 && !col)) return SG_EINVAL;
  // connected components (every stored entry an undirected edge): union-find
  std::vector<int64_t> p((size_t)n);
  std::iota(p.begin(), p.end(), 0);
  for (int64_t u = 0; u < n; ++u) {
    if (row_ptr[u + 1] < row_ptr[u] || row_ptr[u + 1] > nnz) return SG_EINVAL;
    for (int64_t e = row_ptr[u]; e < row_ptr[u + 1]; ++e) {
      const int64_t v = col[e];
      if (v < 0 || v >= n) return SG_EINVAL;
      int64_t a = find_root(p, u), b = find_root(p, v);
      if (a != b) p[(size_t)std::max(a, b)] = std::min(a, b);
    }
  }
  // component weights sum(deg + kappa), heaviest first onto the lightest shard
  std::vector<int64_t> root((size_t)n), weight((size_t)n, 0);
  for (int64_t u = 0; u < n; ++u) {
    root[(size_t)u] = find_root(p, u);
    weight[(size_t)root[(size_t)u]] += (row_ptr[u + 1] - row_ptr[u]) + kappa;
  }
  std::vector<int64_t> comps;
  for (int64_t u = 0; u < n; ++u)
    if (root[(size_t)u] == u) comps.push_back(u);
  std::stable_sort(comps.begin(), comps.end(), [&](int64_t a, int64_t b) {
    return weight[(size_t)a] > weight[(size_t)b];
  });
  using Slot = std::pair<int64_t, int32_t>;                     // (load, shard)
  std::priority_queue<Slot, std::vector<Slot>, std::greater<Slot>> pq;
  for (int32_t r = 0; r < world; ++r) pq.push({0, r});
  std::vector<int32_t> shard_of_root((size_t)n, 0);
  std::vector<int64_t> ld((size_t)world, 0);
  for (int64_t c : comps) {
    Slot s = pq.top();
    pq.pop();
    shard_of_root[(size_t)c] = s.second;
    s.first += weight[(size_t)c];
    ld[(size_t)s.second] = s.first;
    pq.push(s);
  }
  for (int64_t u = 0; u < n; ++u) shard[u] = shard_of_root[(size_t)root[(size_t)u]];
  if (load)
    for (int32_t r = 0; r < world; ++r) load[r] = ld[(size_t)r];
  return SG_OK;
}

sg_status sg_shard_csr(int64_t n, const int64_t *row_ptr, const int32_t *col, const int32_t *shard,
                       int32_t r, int64_t *row_ptr_out, int32_t *col_out, int64_t *nnz_out) {
  if (n < 0 || (n > 0 && (!row_ptr || !shard)) || !nnz_out) return SG_EINVAL;
  int64_t cnt = 0;
  for (int64_t u = 0; u < n; ++u)
    if (shard[u] == r) cnt += row_ptr[u + 1] - row_ptr[u];
  *nnz_out = cnt;
  if (!row_ptr_out && !col_out) return SG_OK;
  if (!row_ptr_out || (cnt > 0 && !col_out)) return SG_EINVAL;
  int64_t o = 0;
  row_ptr_out[0] = 0;
  for (int64_t u = 0; u < n; ++u) {
    if (shard[u] == r) {
      for (int64_t e = row_ptr[u]; e < row_ptr[u + 1]; ++e) col_out[o++] = col[e];
    }
    row_ptr_out[u + 1] = o;
  }
  return SG_OK;
}

sg_status sg_merge_shard_labels(int64_t n, const int32_t *shard, int32_t world, const int32_t *labels,
                                int32_t *out) {
  if (n < 0 || world < 1 || (n > 0 && (!shard || !labels || !out))) return SG_EINVAL;
  for (int64_t v = 0; v < n; ++v) {
    const int32_t r = shard[v];
    if (r < 0 || r >= world) return SG_EINVAL;
    out[v] = labels[(int64_t)r * n + v];
  }
  return SG_OK;
}

}  // extern "C"
