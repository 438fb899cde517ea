// internal.h — shared declarations of libgcsm (product side).
// Device/host data layout:
//   VDesc  per vertex, 16 B, in HBM: where the vertex's *main* list lives
//          (HBM cache slot or mapped pinned host memory — one generic
//          pointer, UVA), its length, and its delta record (updated vertices).
//   DRec   per updated vertex x ∈ U: offsets of ins(x) / del(x) in the
//          device delta list. For x ∈ U the main list is the stable part
//          N_S(x) = N(x) \ del(x); views: S = main, OLD (N) = main ∪ del,
//          NEW (N') = main ∪ ins (SURVEY §8 notation; "N' = N ∪ ΔN").
//   Unit   one level-1 node: term i, kind ±, oriented seed (a, b).
#pragma once
#include <cstdint>
#include <cstddef>
#include <algorithm>
#include <atomic>
#include <chrono>
#include <functional>
#include <string>
#include <thread>
#include <vector>

#define GCSM_MAXK 8
#define GCSM_MAXM 28
#define GCSM_MAXPLANS (2 * GCSM_MAXM)
#define GCSM_MAX_PEERS 7     // linked peer contexts whose HBM caches a context reads (gcsm_link_peers)
#define GCSM_MAX_QUERIES 32  // standing queries per context (gcsm_add_query; all 29 connected 3-5-vertex motifs fit)

namespace gcsm {

enum View : int8_t { VIEW_S = 0, VIEW_OLD = 1, VIEW_NEW = 2 };

struct alignas(16) VDesc {
  const int32_t *ptr;  // main list (device-visible address: HBM cache or mapped host)
  uint32_t len;        // main list length
  uint32_t upd;        // 0, or 1 + index of the vertex's DRec (x ∈ U)
};
static_assert(sizeof(VDesc) == 16, "VDesc must be 16 bytes");

struct alignas(16) DRec {
  uint32_t ins_off, ins_len, del_off, del_len;  // into the device delta list
};

struct alignas(16) Unit {
  int32_t a, b;   // f(order[0]) = a, f(order[1]) = b
  int32_t plan;   // 2 * term + kind (kind 0 = insertion "+", 1 = deletion "-")
  int32_t pad;
};

// One term position (a "loop level" of Fig. 2): candidates for order[p] are
// the intersection of the views of the backward neighbours' lists.
struct LevelPlan {
  int8_t nb;           // number of backward lists
  int8_t bpos[7];      // their term positions
  int8_t bview[7];     // their views (View)
  int8_t reuse;        // -1, or an earlier position p' >= 2 whose candidate set
                       // (same label, lists ⊆ these lists) is the driver (code motion)
  int8_t nrest;        // lists not covered by the reused set
  int8_t rest[7];      // indices into bpos/bview
  int8_t ninj;         // matched positions to exclude (not backward neighbours)
  int8_t inj[7];
  int8_t nlo, lo[7];   // symmetry breaking: f(order[p]) > f(position lo[i])
  int8_t nhi, hi[7];   //                    f(order[p]) < f(position hi[i])
  int8_t fmask;        // position 4 (k >= 5) only, when position 3 is one of its backward neighbours: the backward
                       // lists at positions <= 2 (bit b); their intersection F is fixed per level-2 entry and every
                       // level-3 node whose list misses F has no position-4 candidate (lane-parallel filter)
  int8_t f3;           // index b of position 3 among the backward lists (with fmask)
  int8_t hmask;        // last position (k >= 5) only: backward lists (bit b = bpos[b]) whose positions are <= 2,
                       // i.e. fixed once a level-2 partial match is chosen; their intersection is hoisted to the
                       // level-2 entry (loop-invariant code motion): empty -> the entry's subtree holds no match
  int32_t label;       // required data label of order[p], -1 = any
};

struct DevPlan {
  int32_t k;
  int32_t kind;              // 0 "+", 1 "-"
  int8_t order[GCSM_MAXK];   // query vertex at each term position
  int32_t label0, label1;    // labels of the seed endpoints (-1 = any)
  int32_t seed_rel;          // symmetry breaking on the seed: 0 none, 1 f(order[0]) < f(order[1]), 2 >
  LevelPlan lv[GCSM_MAXK];   // valid for positions 2..k-1
};

// ------------------------------------------------------------ host utilities
struct Timer {
  std::chrono::steady_clock::time_point t0 = std::chrono::steady_clock::now();
  double ms() const {
    return std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
  }
};

// Persistent host worker pool (one per process): spawning std::threads per
// call cost ~1 ms per parallel region on the 16-core box; the pool wakes
// parked workers instead. run() executes fn(tid) for tid in [0, nthreads),
// the caller being tid 0; calls from different host threads are serialised.
void pool_run(int nthreads, const std::function<void(int)> &fn);
int pool_size();

// Static-partitioned parallel for over [0, n).
inline void parallel_for(int threads, int64_t n, const std::function<void(int, int64_t, int64_t)> &fn) {
  if (n <= 0) return;
  const int t = (int)std::min<int64_t>(std::min(threads, pool_size()), n);
  if (t <= 1) {
    fn(0, 0, n);
    return;
  }
  pool_run(t, [&](int i) { fn(i, n * i / t, n * (i + 1) / t); });
}

// Dynamic (atomic cursor) parallel for, chunked.
inline void parallel_dyn(int threads, int64_t n, int64_t chunk, const std::function<void(int, int64_t)> &fn) {
  if (n <= 0) return;
  std::atomic<int64_t> next{0};
  const int t = (int)std::max<int64_t>(1, std::min<int64_t>(std::min(threads, pool_size()), (n + chunk - 1) / chunk));
  pool_run(t, [&](int tid) {
    for (;;) {
      const int64_t s = next.fetch_add(chunk);
      if (s >= n) break;
      const int64_t e = std::min(n, s + chunk);
      for (int64_t i = s; i < e; ++i) fn(tid, i);
    }
  });
}

// Parallel merge sort on the worker pool (no OpenMP: its spinning team would
// compete with the pool for the cores). Stable if `stable`.
template <typename T, typename Cmp>
void parallel_sort(std::vector<T> &v, Cmp cmp, int threads, bool stable = false) {
  const int64_t n = (int64_t)v.size();
  int t = 1;
  while (t * 2 <= threads && n / (t * 2) >= 4096) t *= 2;
  if (t == 1) {
    if (stable) std::stable_sort(v.begin(), v.end(), cmp);
    else std::sort(v.begin(), v.end(), cmp);
    return;
  }
  std::vector<int64_t> cut(t + 1);
  for (int i = 0; i <= t; ++i) cut[i] = n * i / t;
  parallel_for(t, t, [&](int, int64_t lo, int64_t hi) {
    for (int64_t i = lo; i < hi; ++i) {
      if (stable) std::stable_sort(v.begin() + cut[i], v.begin() + cut[i + 1], cmp);
      else std::sort(v.begin() + cut[i], v.begin() + cut[i + 1], cmp);
    }
  });
  std::vector<T> tmp(v.size());
  std::vector<T> *src = &v, *dst = &tmp;
  for (int w = 1; w < t; w *= 2) {
    const int pairs = t / (2 * w);
    parallel_for(pairs, pairs, [&](int, int64_t lo, int64_t hi) {
      for (int64_t p = lo; p < hi; ++p) {
        const int64_t a = cut[2 * w * p], b = cut[2 * w * p + w], c = cut[2 * w * (p + 1)];
        std::merge(src->begin() + a, src->begin() + b, src->begin() + b, src->begin() + c, dst->begin() + a, cmp);
      }
    });
    std::swap(src, dst);
  }
  if (src != &v) v.swap(tmp);
}

// ------------------------------------------------------------ plan (plan.cpp)
struct QueryPlan {
  int k = 0, m = 0;
  int qe[GCSM_MAXM][2];         // numbered query edges R_1..R_m (R12), (pos-min, pos-max) endpoints
  int qlab[GCSM_MAXK];          // -1 = any
  bool labelled = false;
  uint64_t automorphisms = 0;
  bool symmetry = false;                        // restrictions below are active in `plans`
  std::vector<std::pair<int, int>> restrictions;  // (u, w): f(u) < f(w) selects one embedding per Aut_L orbit
  std::vector<DevPlan> plans;   // 2*m: index 2*term + kind
};

// Returns "" on success, else the EINVAL reason.
// symmetry: add the symmetry-breaking restrictions of Aut_L(Q) (counts then scale by |Aut_L|)
std::string build_plan(int k, int m, const int32_t *qedges, const int32_t *qlabels, const int32_t *order,
                       QueryPlan &out, bool symmetry = false);

// ------------------------------------------------------------ RNG (estimator.cpp)
uint64_t rng_mix(uint64_t z);
uint64_t rng_chain(uint64_t h, uint64_t x);
int64_t binomial(uint64_t key, int64_t n, double p);

// ------------------------------------------------------------ sharding
void shard_lpt(int64_t n, const uint64_t *cost, int world, int32_t *rank_out, int threads = 1,
               std::vector<size_t> *order_out = nullptr);

}  // namespace gcsm
