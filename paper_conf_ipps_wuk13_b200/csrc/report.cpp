// report.cpp — host-side Phase III (approach 2) and the hash-pair stream.
//
// Phase III: "initialize a union-find data structure
// of size n ... enumerate all connected components in G_II and for each
// connected component, perform a union of the set of all vertices in G that
// constitute the first- and second-level shingles of that component".
// A component of G_II is connected through shared S1' nodes, so uniting, for
// every G_II group h, the constituents of h and of all its S1' members yields
// exactly the per-component unions.  Constituents of an exact (s <= 2) id are
// recovered algebraically, v = (h - B) * A^(P-2) mod P (A_j invertible since
// A_j != 0 mod P); for s >= 3 they are recomputed from the row of
// the smallest generator (AMB-18).
#include "report.h"

#include <algorithm>
#include <cstring>

namespace sg {

namespace {

constexpr uint64_t P = 0x7FFFFFFFull;

uint64_t mix(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ull;
  z = (z ^ (z >> 27)) * 0x94d049bb133111ebull;
  return z ^ (z >> 31);
}

uint64_t powmod(uint64_t b, uint64_t e) {
  uint64_t r = 1;
  b %= P;
  while (e) {
    if (e & 1) r = r * b % P;
    b = b * b % P;
    e >>= 1;
  }
  return r;
}

struct UF {
  std::vector<int64_t> p;
  explicit UF(int64_t n) : p((size_t)n) {
    for (int64_t i = 0; i < n; ++i) p[(size_t)i] = i;
  }
  int64_t find(int64_t x) {
    int64_t r = x;
    while (p[(size_t)r] != r) r = p[(size_t)r];
    while (p[(size_t)x] != r) {
      int64_t nx = p[(size_t)x];
      p[(size_t)x] = r;
      x = nx;
    }
    return r;
  }
  void unite(int64_t a, int64_t b) {
    a = find(a);
    b = find(b);
    if (a == b) return;
    if (a < b) p[(size_t)b] = a;
    else p[(size_t)a] = b;
  }
};

// top-s vertex ids of a row under (A, B), ascending by hash
void top_s_vertices(const uint32_t *row, int64_t len, int s, uint32_t A, uint32_t B,
                    std::vector<uint32_t> &out) {
  std::vector<std::pair<uint32_t, uint32_t>> best;  // (hash, vertex)
  best.reserve((size_t)s + 1);
  for (int64_t e = 0; e < len; ++e) {
    uint32_t v = row[e];
    uint32_t h = (uint32_t)(((uint64_t)A * v + B) % P);
    if ((int)best.size() == s && h >= best.back().first) continue;
    auto it = std::lower_bound(best.begin(), best.end(), std::make_pair(h, v));
    best.insert(it, std::make_pair(h, v));
    if ((int)best.size() > s) best.pop_back();
  }
  out.clear();
  for (auto &x : best) out.push_back(x.second);
}

void decode_exact(uint64_t id, int s, uint32_t A, uint32_t B, std::vector<uint32_t> &out) {
  uint64_t Ainv = powmod(A, P - 2);
  uint64_t hs[2];
  int k = 0;
  if (s == 1) {
    hs[k++] = id;
  } else {
    hs[k++] = id >> 31;
    hs[k++] = id & P;
  }
  out.clear();
  for (int i = 0; i < k; ++i) out.push_back((uint32_t)(((hs[i] + P - B) % P) * Ainv % P));
}

}  // namespace

void hash_pairs(uint64_t seed, int32_t c, uint32_t *A, uint32_t *B) {
  uint64_t state = seed;
  for (int32_t j = 0; j < c; ++j) {
    state += 0x9E3779B97F4A7C15ull;
    A[j] = (uint32_t)(1 + mix(state) % (P - 1));
    state += 0x9E3779B97F4A7C15ull;
    B[j] = (uint32_t)(mix(state) % P);
  }
}

int64_t report_host(const ReportInput &in, int32_t mode, int32_t min_size, int32_t *labels) {
  UF uf(in.n);
  std::vector<uint32_t> cons, tmp;
  // constituents / generators of first-level node k
  auto first_level = [&](int64_t k, std::vector<uint32_t> &out) {
    out.clear();
    const uint32_t *L = in.lmem + in.loff[k];
    const int64_t len = in.loff[k + 1] - in.loff[k];
    if (mode == 1) {
      out.assign(L, L + len);
      return;
    }
    const int j = in.trial1[k];
    if (in.s1 <= 2) {
      decode_exact(in.id1[k], in.s1, in.A1[j], in.B1[j], out);
    } else {
      const uint32_t u = L[0];  // smallest generator
      top_s_vertices(reinterpret_cast<const uint32_t *>(in.col + in.row_ptr[u]),
                     in.row_ptr[u + 1] - in.row_ptr[u], in.s1, in.A1[j], in.B1[j], out);
    }
  };
  for (int64_t h = 0; h < in.nh; ++h) {
    const uint32_t *K = in.kmem + in.koff[h];
    const int64_t nK = in.koff[h + 1] - in.koff[h];
    int64_t anchor = -1;
    auto add = [&](const std::vector<uint32_t> &vs) {
      for (uint32_t v : vs) {
        if (anchor < 0) anchor = v;
        else uf.unite(anchor, v);
      }
    };
    if (mode == 0) {
      const int t = in.trial2[h];
      if (in.s2 <= 2) {
        decode_exact(in.id2[h], in.s2, in.A2[t], in.B2[t], cons);
      } else {
        const int64_t kmin = K[0];
        top_s_vertices(in.lmem + in.loff[kmin], in.loff[kmin + 1] - in.loff[kmin], in.s2,
                       in.A2[t], in.B2[t], cons);
      }
      add(cons);
    }
    for (int64_t i = 0; i < nK; ++i) {
      first_level(K[i], tmp);
      add(tmp);
    }
  }
  std::vector<int64_t> size((size_t)in.n, 0);
  for (int64_t v = 0; v < in.n; ++v) size[(size_t)uf.find(v)]++;
  const int64_t thr = std::max<int64_t>(2, min_size);
  int64_t nc = 0;
  for (int64_t v = 0; v < in.n; ++v) {
    const int64_t r = uf.find(v);
    if (labels) labels[v] = size[(size_t)r] >= min_size ? (int32_t)r : (int32_t)v;
    if (r == v && size[(size_t)r] >= thr) ++nc;
  }
  return nc;
}

}  // namespace sg
