// gcsm_inputs/gen.cpp — seeded synthetic input generators.
//
// Shared by the product tests/bench AND the oracle tests: this module holds
// none of the method's arithmetic (no matching, no estimator, no caching).
// It only produces inputs shaped like the paper's workloads:
//   * R-MAT graphs (recursive-matrix edge sampler), symmetrised, loop-free,
//     deduplicated, vertex ids permuted with a seeded permutation
//     (SURVEY §8d "Configs as concrete synthetic inputs");
//   * vertex labels uniform over L values;
//   * the update-stream protocol of PAPER.md P:331 (sample edges uniformly
//     without replacement, mark each + or - with p = 1/2; G_0 drops the
//     insertion-marked edges).
// Every random draw is a pure function of (seed, counter) through splitmix64,
// so the output is identical for any thread count and on any host.
#include <algorithm>
#include <cstdint>
#include <cstring>
#include <numeric>
#include <unordered_map>
#include <vector>
#include <parallel/algorithm>
#include <omp.h>
#include <chrono>
#include <cstdio>
#include <cstdlib>

static double gi_now() {
  return std::chrono::duration<double>(std::chrono::steady_clock::now().time_since_epoch()).count();
}
#define GI_T(label) do { if (std::getenv("GI_TIMING")) std::fprintf(stderr, "[gi] %s %.2f s\n", label, gi_now() - t_start); } while (0)

namespace {

inline uint64_t sm64(uint64_t z) {
  z += 0x9E3779B97F4A7C15ULL;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}
inline uint64_t h2(uint64_t a, uint64_t b) { return sm64(a ^ sm64(b)); }
inline double u01(uint64_t x) { return (double)(x >> 11) * (1.0 / 9007199254740992.0); }

struct Cand {
  uint64_t key;  // (u << 32) | v with u < v
  int64_t idx;   // generation index (earlier wins)
};

// Integer thresholds of the R-MAT quadrant test: u01(x) < t  <=>  (x >> 11) < ceil(t * 2^53) (x >> 11 is an
// integer below 2^53 and the scaling by 2^-53 is exact), so the draws are the same as comparing doubles.
struct RmatT {
  uint64_t ta, tab, tabc;
  uint64_t lvl[64];  // sm64(l + 1): the per-level half of h2(base, l + 1)
};
inline uint64_t ceil53(double t) {
  const double x = t * 9007199254740992.0;
  const uint64_t f = (uint64_t)x;
  return (double)f == x ? f : f + 1;
}
inline RmatT rmat_thresholds(double a, double b, double c, int scale) {
  RmatT T;
  T.ta = ceil53(a);
  T.tab = ceil53(a + b);
  T.tabc = ceil53(a + b + c);
  for (int l = 0; l < scale && l < 64; ++l) T.lvl[l] = sm64((uint64_t)l + 1);
  return T;
}

// One R-MAT draw for candidate index j. Returns false for self loops / rejected ids.
inline bool rmat_one(int scale, const RmatT& T, uint64_t seed, int64_t j, int64_t id_limit, uint64_t* key) {
  uint64_t u = 0, v = 0;
  const uint64_t base = h2(seed, (uint64_t)j);
  for (int l = 0; l < scale; ++l) {
    const uint64_t z = sm64(base ^ T.lvl[l]) >> 11;  // h2(base, l + 1)
    const uint64_t ge_a = z >= T.ta, ge_ab = z >= T.tab, ge_abc = z >= T.tabc;
    u = (u << 1) | ge_ab;                          // quadrants c, d
    v = (v << 1) | ((ge_a & (1 - ge_ab)) | ge_abc);  // quadrants b, d
  }
  if (u == v) return false;
  if (id_limit > 0 && ((int64_t)u >= id_limit || (int64_t)v >= id_limit)) return false;
  if (u > v) std::swap(u, v);
  *key = (u << 32) | v;
  return true;
}

// Parallel sort of candidates by (key, idx) or by idx: one MSD pass into 2^bits buckets by the top bits of the
// sort field (counting sort over thread-local histograms), then each bucket sorted on its own.
template <bool BY_KEY>
void bucket_sort(std::vector<Cand>& v, int bits, uint64_t maxval) {
  const int64_t n = (int64_t)v.size();
  if (n < (1 << 16)) {
    if (BY_KEY) std::sort(v.begin(), v.end(), [](const Cand& x, const Cand& y) {
      return x.key < y.key || (x.key == y.key && x.idx < y.idx); });
    else std::sort(v.begin(), v.end(), [](const Cand& x, const Cand& y) { return x.idx < y.idx; });
    return;
  }
  int shift = 0;
  while (shift < 64 && (maxval >> shift) >= (1ull << bits)) ++shift;
  const int nb = 1 << bits;
  const int nt = omp_get_max_threads();
  std::vector<int64_t> hist((size_t)nt * nb, 0);
  auto field = [&](const Cand& c) -> uint64_t { return BY_KEY ? c.key : (uint64_t)c.idx; };
#pragma omp parallel
  {
    const int t = omp_get_thread_num();
    const int64_t lo = n * t / nt, hi = n * (t + 1) / nt;
    int64_t* h = &hist[(size_t)t * nb];
    for (int64_t i = lo; i < hi; ++i) h[field(v[i]) >> shift]++;
  }
  std::vector<int64_t> start((size_t)nb + 1, 0);
  {  // bucket-major, thread-minor exclusive scan (a stable scatter)
    int64_t run = 0;
    for (int bkt = 0; bkt < nb; ++bkt) {
      start[bkt] = run;
      for (int t = 0; t < nt; ++t) {
        const int64_t c = hist[(size_t)t * nb + bkt];
        hist[(size_t)t * nb + bkt] = run;
        run += c;
      }
    }
    start[nb] = run;
  }
  std::vector<Cand> out((size_t)n);
#pragma omp parallel
  {
    const int t = omp_get_thread_num();
    const int64_t lo = n * t / nt, hi = n * (t + 1) / nt;
    int64_t* h = &hist[(size_t)t * nb];
    for (int64_t i = lo; i < hi; ++i) out[(size_t)h[field(v[i]) >> shift]++] = v[i];
  }
#pragma omp parallel for schedule(dynamic, 1)
  for (int bkt = 0; bkt < nb; ++bkt) {
    auto b0 = out.begin() + start[bkt], b1 = out.begin() + start[bkt + 1];
    if (BY_KEY) std::sort(b0, b1, [](const Cand& x, const Cand& y) {
      return x.key < y.key || (x.key == y.key && x.idx < y.idx); });
    else std::sort(b0, b1, [](const Cand& x, const Cand& y) { return x.idx < y.idx; });
  }
  v.swap(out);
}

}  // namespace

extern "C" {

// Exactly n_edges unique undirected edges of an R-MAT(scale; a,b,c,d=1-a-b-c)
// graph: candidates are drawn in index order, the first n_edges distinct
// non-loop pairs (by generation index) are kept, then the vertex ids are
// relabelled with a seeded uniform permutation of [0, n_ids) where
// n_ids = id_limit > 0 ? id_limit : 2^scale. Output pairs (u<v) in generation
// order. Returns n_edges, or -1 if the id space cannot hold that many edges.
// planted_groups > 0: the candidate stream starts with the edges of that many
// planted cliques of planted_size vertices each (members drawn uniformly from
// the id space, so they come first in generation order and are always kept):
// community structure R-MAT lacks (SURVEY §8d workload-realism note).
int64_t gi_rmat_edges(int32_t scale, int64_t n_edges, double a, double b, double c,
                      uint64_t seed, int64_t id_limit, int32_t threads, int32_t* out_uv,
                      int64_t planted_groups, int32_t planted_size) {
  if (threads > 0) omp_set_num_threads(threads);
  const double t_start = gi_now();
  const RmatT T = rmat_thresholds(a, b, c, scale);
  const int64_t n_ids = id_limit > 0 ? id_limit : (int64_t(1) << scale);
  if ((double)n_edges > 0.5 * (double)n_ids * (double)(n_ids - 1)) return -1;
  std::vector<Cand> cands;
  int64_t next_j = 0;
  int64_t uniq = 0;
  if (planted_groups > 0 && planted_size >= 2) {
    const int64_t per = (int64_t)planted_size * (planted_size - 1) / 2;
    const int64_t np = planted_groups * per;
    cands.resize((size_t)np);
    std::vector<uint8_t> ok((size_t)np);
    const uint64_t gseed = h2(seed, 0x504C414E54ULL);
#pragma omp parallel for schedule(static)
    for (int64_t g = 0; g < planted_groups; ++g) {
      uint64_t mem[64];
      const int sz = planted_size < 64 ? planted_size : 64;
      for (int i = 0; i < sz; ++i) mem[i] = h2(gseed, (uint64_t)(g * sz + i)) % (uint64_t)n_ids;
      int64_t t = g * per;
      for (int i = 0; i < sz; ++i)
        for (int j = i + 1; j < sz; ++j, ++t) {
          uint64_t u = mem[i], v = mem[j];
          ok[t] = u != v;
          if (u > v) std::swap(u, v);
          cands[t] = Cand{(u << 32) | v, t};
        }
    }
    size_t w = 0;
    for (int64_t t = 0; t < np; ++t)
      if (ok[t]) cands[w++] = cands[t];
    cands.resize(w);
    next_j = np;
    bucket_sort<true>(cands, 14, (uint64_t)n_ids << 32);
    size_t o = 0;
    for (size_t i = 0; i < cands.size(); ++i)
      if (o == 0 || cands[i].key != cands[o - 1].key) cands[o++] = cands[i];
    cands.resize(o);
    uniq = (int64_t)o;
  }
  const int64_t rmat_base = next_j;  // R-MAT draw j = generation index - rmat_base (same draws with or without planting)
  while (uniq < n_edges) {
    const int64_t want = (int64_t)((double)(n_edges - uniq) * 1.25) + 1024;
    const size_t old = cands.size();
    cands.resize(old + (size_t)want);
    std::vector<uint8_t> ok((size_t)want);
#pragma omp parallel for schedule(static)
    for (int64_t t = 0; t < want; ++t) {
      uint64_t key = 0;
      ok[t] = rmat_one(scale, T, seed, next_j + t - rmat_base, id_limit, &key);
      cands[old + t] = Cand{key, next_j + t};
    }
    size_t w = old;
    for (int64_t t = 0; t < want; ++t)
      if (ok[t]) cands[w++] = cands[old + t];
    cands.resize(w);
    next_j += want;
    GI_T("draw");
    bucket_sort<true>(cands, 14, (uint64_t)n_ids << 32);
    size_t o = 0;
    for (size_t i = 0; i < cands.size(); ++i)
      if (o == 0 || cands[i].key != cands[o - 1].key) cands[o++] = cands[i];
    cands.resize(o);
    uniq = (int64_t)o;
    GI_T("sort+unique");
  }
  // keep the n_edges earliest by generation index, in generation order
  bucket_sort<false>(cands, 14, (uint64_t)next_j);
  cands.resize((size_t)n_edges);
  GI_T("idx sort");
  // seeded permutation of vertex ids (Fisher-Yates, counter-based draws)
  std::vector<int32_t> perm((size_t)n_ids);
  std::iota(perm.begin(), perm.end(), 0);
  const uint64_t pseed = h2(seed, 0x5045524DULL);
  for (int64_t i = n_ids - 1; i > 0; --i) {
    const uint64_t r = h2(pseed, (uint64_t)i);
    const int64_t j = (int64_t)(r % (uint64_t)(i + 1));
    std::swap(perm[i], perm[j]);
  }
#pragma omp parallel for schedule(static)
  for (int64_t e = 0; e < n_edges; ++e) {
    int32_t u = perm[(size_t)(cands[e].key >> 32)];
    int32_t v = perm[(size_t)(cands[e].key & 0xFFFFFFFFULL)];
    if (u > v) std::swap(u, v);
    out_uv[2 * e] = u;
    out_uv[2 * e + 1] = v;
  }
  return n_edges;
}

// Road-network-shaped graph (RoadNetPA / RoadNetCA of Table I; the motif experiment of Fig. 11,
// every vertex has a small degree): a W x H lattice whose edges are kept with probability p_keep,
// plus one diagonal per cell with probability p_diag (road junctions close triangles), cells in row-major
// order, each cell emitting (right, down, diagonal); then the vertex ids are relabelled with a seeded uniform
// permutation. Writes up to cap pairs (u < v) in generation order; returns the number of edges.
int64_t gi_grid_edges(int32_t W, int32_t H, double p_keep, double p_diag, uint64_t seed, int32_t* out_uv,
                      int64_t cap) {
  const int64_t n = (int64_t)W * H;
  std::vector<int32_t> perm((size_t)n);
  std::iota(perm.begin(), perm.end(), 0);
  const uint64_t pseed = h2(seed, 0x47524944ULL);
  for (int64_t i = n - 1; i > 0; --i) {
    const int64_t j = (int64_t)(h2(pseed, (uint64_t)i) % (uint64_t)(i + 1));
    std::swap(perm[i], perm[j]);
  }
  int64_t m = 0;
  auto emit = [&](int64_t a, int64_t b) {
    if (m < cap) {
      int32_t u = perm[(size_t)a], v = perm[(size_t)b];
      if (u > v) std::swap(u, v);
      out_uv[2 * m] = u;
      out_uv[2 * m + 1] = v;
    }
    ++m;
  };
  for (int64_t y = 0; y < H; ++y)
    for (int64_t x = 0; x < W; ++x) {
      const int64_t c = y * W + x;
      if (x + 1 < W && u01(h2(seed, 3 * (uint64_t)c)) < p_keep) emit(c, c + 1);
      if (y + 1 < H && u01(h2(seed, 3 * (uint64_t)c + 1)) < p_keep) emit(c, c + W);
      if (x + 1 < W && y + 1 < H && u01(h2(seed, 3 * (uint64_t)c + 2)) < p_diag) {
        if (h2(seed ^ 0xD1A6ULL, (uint64_t)c) & 1) emit(c, c + W + 1);
        else emit(c + 1, c + W);
      }
    }
  return m;
}

// Symmetric CSR of an undirected simple edge list (u != v, no duplicates): row_ptr[n+1], col[2m'], each row
// sorted ascending. skip: NULL, or m flags (1 = leave edge e out: the insertion-marked edges of the stream,
// P:331). Parallel: atomic degree counts and slot claims, then per-row sorts. Returns -1 on a bad edge.
int32_t gi_build_csr_skip(int32_t n, int64_t m, const int32_t* uv, const uint8_t* skip, int32_t threads,
                          int64_t* row_ptr, int32_t* col) {
  if (threads > 0) omp_set_num_threads(threads);
  std::vector<int64_t> deg((size_t)n + 1, 0);
  int bad = 0;
#pragma omp parallel for schedule(static) reduction(| : bad)
  for (int64_t e = 0; e < m; ++e) {
    if (skip && skip[e]) continue;
    const int32_t u = uv[2 * e], v = uv[2 * e + 1];
    if (u < 0 || v < 0 || u >= n || v >= n || u == v) {
      bad = 1;
      continue;
    }
    __atomic_fetch_add(&deg[u], 1, __ATOMIC_RELAXED);
    __atomic_fetch_add(&deg[v], 1, __ATOMIC_RELAXED);
  }
  if (bad) return -1;
  row_ptr[0] = 0;
  for (int32_t i = 0; i < n; ++i) row_ptr[i + 1] = row_ptr[i] + deg[i];
  std::vector<int64_t> pos(row_ptr, row_ptr + n);
#pragma omp parallel for schedule(static)
  for (int64_t e = 0; e < m; ++e) {
    if (skip && skip[e]) continue;
    const int32_t u = uv[2 * e], v = uv[2 * e + 1];
    col[__atomic_fetch_add(&pos[u], 1, __ATOMIC_RELAXED)] = v;
    col[__atomic_fetch_add(&pos[v], 1, __ATOMIC_RELAXED)] = u;
  }
#pragma omp parallel for schedule(dynamic, 4096)
  for (int32_t i = 0; i < n; ++i) std::sort(col + row_ptr[i], col + row_ptr[i + 1]);
  return 0;
}

int32_t gi_build_csr(int32_t n, int64_t m, const int32_t* uv, int32_t threads, int64_t* row_ptr, int32_t* col) {
  return gi_build_csr_skip(n, m, uv, nullptr, threads, row_ptr, col);
}

// Labels uniform over [0, L).
void gi_labels(int32_t n, int32_t L, uint64_t seed, int32_t* labels) {
  const uint64_t s = h2(seed, 0x4C4142454CULL);
#pragma omp parallel for schedule(static)
  for (int32_t i = 0; i < n; ++i) labels[i] = (int32_t)(h2(s, (uint64_t)i) % (uint64_t)L);
}

// P:331 stream protocol: n_sample edge indices drawn uniformly without
// replacement from [0, m) in random order (sparse partial Fisher-Yates), each
// marked insertion (sign=+1) or deletion (sign=-1) with p = 1/2.
int64_t gi_stream(int64_t m, int64_t n_sample, uint64_t seed, int64_t* sel, int8_t* sign) {
  if (n_sample > m) return -1;
  std::unordered_map<int64_t, int64_t> swapped;
  swapped.reserve((size_t)n_sample * 2);
  const uint64_t s = h2(seed, 0x53545245414DULL);
  auto at = [&](int64_t i) {
    auto it = swapped.find(i);
    return it == swapped.end() ? i : it->second;
  };
  for (int64_t t = 0; t < n_sample; ++t) {
    const uint64_t r = h2(s, (uint64_t)t);
    const int64_t j = t + (int64_t)(r % (uint64_t)(m - t));
    const int64_t vj = at(j), vt = at(t);
    swapped[j] = vt;
    swapped[t] = vj;
    sel[t] = vj;
    sign[t] = (h2(s ^ 0xABCDEFULL, (uint64_t)t) & 1) ? (int8_t)1 : (int8_t)-1;
  }
  return n_sample;
}

}  // extern "C"
