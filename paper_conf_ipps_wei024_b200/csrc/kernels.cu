// kernels.cu — sm_100a incremental-matching kernels (step ④ of Fig. 3).
//
// What runs: for every level-1 unit (term i of eq. (1), kind ±, oriented seed
// edge (a, b)) the nested loops of Fig. 2b-f extend the
// partial match one query vertex per level; the candidates of a level are the
// intersection of the backward neighbours' lists under their views (DESIGN.md
// R7: S / N / N'), filtered by label and injectivity; the last level only
// counts ("output" -> count).
//
// B200 mapping:
//   * k_level2: warp per unit (dynamic atomic cursor, persistent grid sized to
//     the SM count x occupancy). It computes level 2 (position 2) and either
//     counts (k = 3) or writes the unit's candidate set as one contiguous
//     segment of the level-2 frontier (BFS for the first level).
//   * k_extend: warp per frontier entry (unit, x2): DFS over the remaining
//     levels with per-warp stacks in HBM (180 GB makes D ints per level per
//     warp affordable), code motion (a later level starts from an earlier
//     level's candidate set, STMatch [9] / P:298).
//   * intersections: the 32 lanes take 32 consecutive driver elements
//     (coalesced), each lane probes the other lists by binary search; the
//     warp compacts survivors with ballot/popc. Lists are read through one
//     16-byte descriptor per vertex whose pointer is either the HBM cache
//     slot or the mapped pinned host list (zero-copy): one
//     generic load path, UVA decides the route.
//   * counts: per-warp registers, one 64-bit atomic per warp and counter at
//     the end of the persistent loop.
#include <climits>
#include <cstdio>

#include "kernels.cuh"
#include "stage.cuh"

namespace gcsm {

namespace {

constexpr int kWarps = 8;
constexpr int kBlock = 32 * kWarps;
constexpr unsigned kFull = 0xffffffffu;
#ifndef GCSM_SMEM_INTS
#define GCSM_SMEM_INTS 1024
#endif
#ifndef GCSM_PRESTAGE_MERGE
#define GCSM_PRESTAGE_MERGE 0
#endif
#ifndef GCSM_PIN_SMEM_MAX
#define GCSM_PIN_SMEM_MAX 768  // largest x2 list (ints) pinned in the shared slice; larger ones go to HBM scratch
#endif
#ifndef GCSM_BM_INTS
#define GCSM_BM_INTS 0  // per-warp membership bitmap of the run x2 list; measured slower than merge on C2 (off)
#endif
#ifndef GCSM_COLD_NOINLINE
#define GCSM_COLD_NOINLINE 0  // 1: generic intersection / staging / probe helpers out of line (register pressure)
#endif
#if GCSM_COLD_NOINLINE
#define GCSM_COLD __noinline__
#else
#define GCSM_COLD __forceinline__
#endif
#ifndef GCSM_MINBLOCKS
#define GCSM_MINBLOCKS 4  // resident 256-thread blocks per SM requested from ptxas for k_extend
#endif
constexpr uint32_t kSmemInts = GCSM_SMEM_INTS;  // per-warp shared staging slice
constexpr int kSmemBytes = kWarps * kSmemInts * 4;
#ifndef GCSM_EXT_CHUNK
#define GCSM_EXT_CHUNK 32
#endif
constexpr int kChunk = GCSM_EXT_CHUNK;  // frontier entries per k_extend work grab
#ifndef GCSM_L4_GRAB
#define GCSM_L4_GRAB 64  // k_last4: frontier entries per work grab (processed in rounds of 32)
#endif
#ifndef GCSM_SPLIT_MIN
#define GCSM_SPLIT_MIN 8
#endif
#ifndef GCSM_TASK_SIZE
#define GCSM_TASK_SIZE 2
#endif
constexpr uint32_t kSplitMin = GCSM_SPLIT_MIN;  // level-3 sets larger than this are shared as tasks (k >= 5)
#ifndef GCSM_FSPLIT_MIN
#define GCSM_FSPLIT_MIN 64
#endif
#ifndef GCSM_FTASK_SIZE
#define GCSM_FTASK_SIZE 32
#endif
// level-3 sets larger than kFSplitMin are shared BEFORE the level-3 filter, in slices of kFTaskSize nodes that the
// takers filter themselves (the filter, one lane per node, is the heavy part of a hub entry)
constexpr uint32_t kFSplitMin = GCSM_FSPLIT_MIN, kFTaskSize = GCSM_FTASK_SIZE;
constexpr uint32_t kTaskFilter = 0xffffffffu;  // Task::pad: the slice is unfiltered
#ifndef GCSM_FILT_LANE
#define GCSM_FILT_LANE 128
#endif
constexpr uint32_t kFiltLane = GCSM_FILT_LANE;  // level-3 filter: larger per-node tests run warp-wide
constexpr uint32_t kTaskSize = GCSM_TASK_SIZE;  // level-3 candidates per task

struct LRef {
  const int32_t *m;  // main list
  uint32_t ml;
  const int32_t *x;  // delta segment (ins or del), device memory
  uint32_t xl;
  bool dev;          // main list is in device memory (HBM cache, a staged copy, or shared memory)
};

// Per-warp accumulators: the counts in registers; the byte statistics (warp-uniform values, updated by lane 0)
// in a per-warp block of shared memory, so that they cost no registers in the register-bound kernels.
enum : int { kSHit, kSMiss, kSDelta, kSCopied, kSFill, kSLists, kSSHit, kSPeer, kSN };
struct Acc {
  unsigned long long add = 0, rem = 0;
  unsigned long long *s = nullptr;  // kSN counters (shared memory, this warp's)
  bool l0 = false;
  __device__ __forceinline__ void init(unsigned long long *blk, int lane) {
    s = blk;
    l0 = lane == 0;
    __syncwarp();
    if (l0)
      for (int i = 0; i < kSN; ++i) s[i] = 0;
    __syncwarp();
  }
  __device__ __forceinline__ void stat(int i, unsigned long long v) {
    if (l0) s[i] += v;
  }
};

// NVLink peer cache (NEXT-3): vertex v's main list in a linked peer's HBM cache for this batch, or nullptr. The
// peers apply the same batches, so for v not updated by the batch (upd == 0) their copy of base(v) is ours; a
// peer's descriptors and cache are final before this batch's kernels start and stay until they finish
// (gcsm_link_peers).
__device__ __forceinline__ const int32_t *peer_lookup(const MatchArgs &A, int32_t v, uint32_t ml) {
  for (int p = 0; p < A.npeer; ++p) {
    const int4 raw = __ldg(reinterpret_cast<const int4 *>(A.peer_vdesc[p] + v));
    const char *q = reinterpret_cast<const char *>((unsigned long long)(unsigned)raw.x |
                                                   ((unsigned long long)(unsigned)raw.y << 32));
    if (q >= A.peer_lo[p] && q < A.peer_hi[p] && (uint32_t)raw.z == ml && raw.w == 0)
      return reinterpret_cast<const int32_t *>(A.peer_map[p] + (q - A.peer_lo[p]));
  }
  return nullptr;
}

__device__ __forceinline__ const int32_t *stage_resolve(const MatchArgs &A, int32_t v, const int32_t *hp, uint32_t ml,
                                                        Acc &acc, int lane) {
  const StageRef R{A.stage_state, A.stage_arena, A.stage_cap, A.stage_bump, A.stage_epoch};
  const StageRes r = stage_fetch(R, v, hp, ml, lane);
  if (r.how == kStFilled) {
    acc.stat(kSFill, 4ull * ml);
    acc.stat(kSLists, 1);
  } else if (r.how == kStServed) {
    acc.stat(kSSHit, 4ull * ml);
  }
  return r.p;
}

__device__ __forceinline__ void mark_touched(const MatchArgs &A, int32_t v) {
  if (A.touched) atomicOr(A.touched + (v >> 5), 1u << (v & 31));
}

// Persistent per-warp copy of one vertex's main list (the position-2 vertex x2 of a run of frontier entries
// grouped by x2): `v` = -1 when empty.
struct Pinned {
  int32_t v = -1;
  const int32_t *p = nullptr;
  int32_t bm_v = -1;  // vertex whose main list is in the warp's bitmap (the run's x2), -1 = none
  int32_t rv = -1;    // vertex whose descriptor is cached in `raw` (the run's x2: no reload per entry)
  int4 raw;
};

__device__ __forceinline__ LRef list_of(const MatchArgs &A, int32_t v, int view, Acc &acc, int lane,
                                        const Pinned &pin = Pinned()) {
  const int4 raw = v == pin.rv ? pin.raw : __ldg(reinterpret_cast<const int4 *>(A.vdesc + v));
  LRef r;
  r.m = reinterpret_cast<const int32_t *>((unsigned long long)(unsigned)raw.x |
                                          ((unsigned long long)(unsigned)raw.y << 32));
  r.ml = (uint32_t)raw.z;
  r.x = nullptr;
  r.xl = 0;
  const uint32_t upd = (uint32_t)raw.w;
  if (upd != 0 && view != VIEW_S) {
    const int4 e = __ldg(reinterpret_cast<const int4 *>(A.drec + (upd - 1)));
    if (view == VIEW_NEW) {
      r.x = A.dlist + e.x;
      r.xl = (uint32_t)e.y;
    } else {
      r.x = A.dlist + e.z;
      r.xl = (uint32_t)e.w;
    }
  }
  const char *p = reinterpret_cast<const char *>(r.m);
  const bool in_cache = p >= A.cache_lo && p < A.cache_hi, in_ubuf = p >= A.ubuf_lo && p < A.ubuf_hi;
  r.dev = in_cache || in_ubuf;
  if (in_cache) acc.stat(kSHit, 4ull * r.ml);
  else if (in_ubuf) acc.stat(kSDelta, 4ull * r.ml);  // the batch's uploaded stable lists of U (device-resident deltas)
  else acc.stat(kSMiss, 4ull * r.ml);
  acc.stat(kSDelta, 4ull * r.xl);
  if (lane == 0) mark_touched(A, v);
  if (v == pin.v) {  // served from this warp's staged copy
    r.m = pin.p;
    r.dev = true;
  } else if (!r.dev && A.npeer && (uint32_t)raw.w == 0 && r.ml > 0) {  // a peer's HBM cache, then the arena
    const int32_t *q = peer_lookup(A, v, r.ml);
    if (q) {
      r.m = q;
      r.dev = true;
      acc.stat(kSPeer, 4ull * r.ml);
    }
  }
  if (!r.dev && A.stage_state && r.ml >= A.stage_min) {  // fetched once per batch into HBM
    r.m = stage_resolve(A, v, r.m, r.ml, acc, lane);
    r.dev = reinterpret_cast<const char *>(r.m) != p;
  }
  return r;
}

__device__ __forceinline__ bool bsearch_has(const int32_t *a, uint32_t n, int32_t v) {
  uint32_t lo = 0, hi = n;
  while (lo < hi) {
    const uint32_t mid = (lo + hi) >> 1;
    if (a[mid] < v) lo = mid + 1;
    else hi = mid;
  }
  return lo < n && a[lo] == v;
}

__device__ __forceinline__ bool contains(const LRef &L, int32_t v) {
  return bsearch_has(L.m, L.ml, v) || (L.xl != 0 && bsearch_has(L.x, L.xl, v));
}

__device__ __forceinline__ uint32_t lb_idx(const int32_t *a, uint32_t n, int32_t v) {  // first i with a[i] >= v
  uint32_t lo = 0, hi = n;
  while (lo < hi) {
    const uint32_t mid = (lo + hi) >> 1;
    if (a[mid] < v) lo = mid + 1;
    else hi = mid;
  }
  return lo;
}

// Two-list intersection by merge path (both lists device-resident, single sorted runs): the warp splits the merged
// sequence a ∪ b into 32 diagonal ranges (co-rank search) and each lane merges its own, O((na + nb) / 32) steps
// instead of ceil(na / 32) rounds of log2(nb)-step binary searches — what a hub entry needs when its lists have
// comparable lengths (C4: one warp intersecting two lists of 10^4-10^5 elements took up to 20 ms by binary search).
// MATERIALIZE: a count pass, an exclusive warp scan of the lanes' counts, and a writing pass keep the output
// sorted. Same survivors as warp_isect (range, exclusions, label).
template <bool MATERIALIZE>
__device__ GCSM_COLD uint32_t merge_isect(const MatchArgs &A, const int32_t *a, uint32_t na, const int32_t *b,
                                          uint32_t nb, const int32_t *excl, int nexcl, int label, int32_t *out,
                                          int lane, int32_t vlo, int32_t vhi) {
  if (vlo != INT_MIN) {
    const uint32_t ua = lb_idx(a, na, vlo + 1), ub = lb_idx(b, nb, vlo + 1);
    a += ua;
    na -= ua;
    b += ub;
    nb -= ub;
  }
  if (vhi != INT_MAX) {
    na = lb_idx(a, na, vhi);
    nb = lb_idx(b, nb, vhi);
  }
  const uint32_t T = na + nb;
  const uint32_t d0 = (uint32_t)(((uint64_t)T * (uint32_t)lane) >> 5);
  const uint32_t d1 = (uint32_t)(((uint64_t)T * (uint32_t)(lane + 1)) >> 5);
  uint32_t lo = d0 > nb ? d0 - nb : 0, hi = d0 < na ? d0 : na;
  while (lo < hi) {
    const uint32_t i = (lo + hi) >> 1;
    if (a[i] <= b[d0 - i - 1]) lo = i + 1;
    else hi = i;
  }
  const uint32_t i0 = lo, j0 = d0 - lo;
  auto pass = [&](bool write, uint32_t base) -> uint32_t {
    uint32_t i = i0, j = j0, c = 0;
    while (i + j < d1) {
      const int32_t ai = i < na ? a[i] : INT_MAX;
      const int32_t bj = j < nb ? b[j] : INT_MAX;
      const bool le = ai <= bj, ge = ai >= bj;
      if (le && ge) {
        bool ok = true;
        for (int e = 0; e < nexcl; ++e) ok = ok && ai != excl[e];
        if (ok && label >= 0) ok = A.lab[ai] == (uint16_t)label;
        if (ok) {
          if (write) out[base + c] = ai;
          ++c;
        }
      }
      i += le;
      j += ge;
    }
    return c;
  };
  const uint32_t c = pass(false, 0);
  uint32_t incl = c;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t y = __shfl_up_sync(kFull, incl, o);
    if (lane >= o) incl += y;
  }
  const uint32_t total = __shfl_sync(kFull, incl, 31);
  if (MATERIALIZE && total) pass(true, incl - c);
  return total;
}

// Warp-cooperative intersection. Driver: the device set dset[0..dn) if dset
// != nullptr (code motion; then every L[] is a probe), else L[drv] (main then
// delta segment; L[drv] is not probed). A driver element v survives if it is
// not any excl[], has the required label, and belongs to every probe list.
// MATERIALIZE: survivors are compacted into out[]. Returns the survivor count
// (warp-uniform).
template <bool MATERIALIZE>
__device__ GCSM_COLD uint32_t warp_isect(const MatchArgs &A, const int32_t *dset, uint32_t dn, const LRef *L,
                                               int nl, int drv, const int32_t *excl, int nexcl, int label,
                                               int32_t *out, int lane, int32_t vlo = INT_MIN, int32_t vhi = INT_MAX) {
  if (!dset && nl == 2 && A.merge2 && L[0].dev && L[1].dev && L[0].xl == 0 && L[1].xl == 0 && L[0].ml && L[1].ml) {
    // two single-run device-resident lists: merge path when cheaper than lane-parallel binary searches
    const uint32_t d = L[drv].ml, big = L[1 - drv].ml;
    const uint32_t lg = 31u - __clz(big | 1u);
    const uint64_t bs_cost = (uint64_t)((d + 31) >> 5) * (7 * lg + 12);
    const uint64_t mg_cost = (MATERIALIZE ? 2ull : 1ull) * (7ull * ((d + big + 31) >> 5)) + 10ull * lg + 40;
    if (mg_cost < bs_cost)
      return merge_isect<MATERIALIZE>(A, L[0].m, L[0].ml, L[1].m, L[1].ml, excl, nexcl, label, out, lane, vlo, vhi);
  }
  const int32_t *s0, *s1;
  uint32_t n0, n1;
  if (dset) {
    s0 = dset; n0 = dn; s1 = nullptr; n1 = 0;
  } else {
    s0 = L[drv].m; n0 = L[drv].ml; s1 = L[drv].x; n1 = L[drv].xl;
  }
  const uint32_t total = n0 + n1;
  uint32_t found = 0;
  for (uint32_t base = 0; base < total; base += 32) {
    const uint32_t i = base + lane;
    bool ok = i < total;
    int32_t v = 0;
    if (ok) v = i < n0 ? s0[i] : s1[i - n0];
    ok = ok && v > vlo && v < vhi;  // symmetry-breaking range
    for (int e = 0; e < nexcl; ++e) ok = ok && v != excl[e];
    if (ok && label >= 0) ok = A.lab[v] == (uint16_t)label;
    for (int p = 0; p < nl; ++p)
      if (ok && (dset || p != drv)) ok = contains(L[p], v);
    const unsigned mask = __ballot_sync(kFull, ok);
    if (MATERIALIZE && ok) out[found + __popc(mask & ((1u << lane) - 1u))] = v;
    found += __popc(mask);
  }
  return found;
}

// device-resident main list: the HBM cache or the batch's uploaded stable lists of U
__device__ __forceinline__ bool is_hit(const MatchArgs &A, const int32_t *p) {
  const char *c = reinterpret_cast<const char *>(p);
  return (c >= A.cache_lo && c < A.cache_hi) || (c >= A.ubuf_lo && c < A.ubuf_hi);
}

// A list already in device memory outside the cache (a warp's staged copy in its HBM scratch).
__device__ __forceinline__ bool is_device(const MatchArgs &A, const int32_t *p) {
  return p >= A.scratch && p < A.scratch_end;
}

// Staging policy: a zero-copy driver list is bulk-copied once
// (full MLP); a probe list is bulk-copied when reading it whole costs no more
// bytes than the probes would (4 L <= 32 B x d x (log2 L - 3): one sector per
// binary-search step below the first 8-int sector), into the warp's shared
// memory slice if it fits, else (zero-copy lists only) into its HBM scratch.
__device__ GCSM_COLD void stage_lists(const MatchArgs &A, LRef *L, int nl, int drv, bool has_set, uint32_t dn,
                                            int32_t *sm, uint32_t sm_cap, int32_t *gbuf, int lane, Acc &acc) {
  const uint32_t d = has_set ? dn : L[drv].ml + L[drv].xl;
  uint32_t sm_used = 0, g_used = 0;
  bool any = false;
  for (int p = 0; p < nl; ++p) {
    const uint32_t n = L[p].ml;
    if (n < 32) continue;
    const bool hit = L[p].dev;
    const bool driver = !has_set && p == drv;
    bool stage;
    const uint32_t lg = 32u - __clz(n);
    if (driver) {
      stage = !hit;
    } else if (hit && A.stage_policy == 1) {
      // device-resident probe list (HBM cache, arena, U lists): latency model — a copy into shared memory costs
      // one dependent round per 512 ints (4 x 16 B per lane in flight), the probes cost one per binary-search step
      // below the last 128-byte line, for every 32 driver elements
      stage = !__isShared(L[p].m) && (n + 511) / 512 <= ((d + 31) / 32) * (lg > 5 ? lg - 5 : 1);
    } else {
      stage = 4ull * n <= 32ull * d * (lg > 4 ? lg - 3 : 1);
    }
    if (!stage) continue;
    const uint32_t n4 = (n + 3) & ~3u;
    if (!hit) acc.stat(kSCopied, 4ull * n);
    if (sm_used + n4 <= sm_cap) {
      warp_copy(sm + sm_used, L[p].m, n, lane);
      L[p].m = sm + sm_used;
      L[p].dev = true;
      sm_used += n4;
      any = true;
    } else if (!hit && g_used + n4 <= 2u * (uint32_t)A.dcap) {
      warp_copy(gbuf + g_used, L[p].m, n, lane);
      L[p].m = gbuf + g_used;
      L[p].dev = true;
      g_used += n4;
      any = true;
    }
  }
  if (any) __syncwarp();
}

// ---- merge-path intersection count (two sorted runs) ------------------------------
// The warp splits the merged sequence a ∪ b into 32 equal diagonal ranges; each lane finds its start by a
// co-rank binary search and merges its range sequentially, counting a[i] == b[j] when it consumes a[i] (ties
// take A first, so an equal pair is counted exactly once even across lane boundaries). O((na+nb)/32 + log)
// instructions per lane instead of ceil(d/32) * log2(L) dependent probes.
// (Runs start anywhere once range-trimmed, so the lanes read scalars; an int4-window variant faulted on trimmed
// runs and was removed.)
__device__ __forceinline__ uint32_t merge_count(const int32_t *a, uint32_t na, const int32_t *b, uint32_t nb,
                                                int label, const uint16_t *lab, int lane) {
  const uint32_t T = na + nb;
  const uint32_t d0 = (uint32_t)(((uint64_t)T * (uint32_t)lane) >> 5);
  const uint32_t d1 = (uint32_t)(((uint64_t)T * (uint32_t)(lane + 1)) >> 5);
  uint32_t lo = d0 > nb ? d0 - nb : 0, hi = d0 < na ? d0 : na;
  while (lo < hi) {
    const uint32_t i = (lo + hi) >> 1;
    if (a[i] <= b[d0 - i - 1]) lo = i + 1;
    else hi = i;
  }
  uint32_t i = lo, j = d0 - lo, cnt = 0;
  // branch-free steps; an equal pair advances both runs (still counted once: the co-rank split puts a[i]
  // before an equal b[j], so the lane owning a[i] counts it and the next lane starts past it)
  while (i + j < d1) {
    const int32_t ai = i < na ? a[i] : INT_MAX;
    const int32_t bj = j < nb ? b[j] : INT_MAX;
    const bool le = ai <= bj, ge = ai >= bj;
    if (le && ge && (label < 0 || lab[ai] == (uint16_t)label)) ++cnt;
    i += le;
    j += ge;
  }
#pragma unroll
  for (int o = 16; o; o >>= 1) cnt += __shfl_xor_sync(kFull, cnt, o);
  return cnt;
}

// lane-parallel count of x[0..nx) present in the sorted list y (label-filtered)
__device__ GCSM_COLD uint32_t probe_count(const int32_t *x, uint32_t nx, const int32_t *y, uint32_t ny, int label,
                                                const uint16_t *lab, int lane, int32_t vlo, int32_t vhi) {
  uint32_t cnt = 0;
  for (uint32_t i = lane; i < nx; i += 32) {
    const int32_t v = x[i];
    if (v > vlo && v < vhi && bsearch_has(y, ny, v) && (label < 0 || lab[v] == (uint16_t)label)) ++cnt;
  }
#pragma unroll
  for (int o = 16; o; o >>= 1) cnt += __shfl_xor_sync(kFull, cnt, o);
  return cnt;
}

__device__ __forceinline__ bool is_host(const MatchArgs &A, const int32_t *p) {
  return !(is_hit(A, p) || is_device(A, p) || __isShared(p));
}

__device__ __forceinline__ uint32_t ilog2(uint32_t x) { return 31u - __clz(x | 1u); }

// Count of the last level for two lists without a reused set: merge path when both main runs are in device
// memory and it is cheaper than per-lane binary search; the tiny delta runs are probed; excluded (matched,
// non-adjacent) vertices that lie in the intersection are subtracted. Returns false if not applicable.
__device__ __forceinline__ bool count2(const MatchArgs &A, const LRef *L, int drv, const int32_t *excl, int nexcl,
                                       int label, int lane, uint32_t *out, int32_t vlo = INT_MIN,
                                       int32_t vhi = INT_MAX) {
  const LRef &X = L[drv], &Y = L[1 - drv];
  if (X.ml < 8 || Y.ml < 8 || !X.dev || !Y.dev) return false;
  const uint32_t d = X.ml + X.xl, big = Y.ml + Y.xl;
  const uint32_t bs_cost = ((d + 31) >> 5) * (7 * ilog2(big) + 12);
  const uint32_t mg_cost = 10 * ilog2(min(X.ml, Y.ml)) + 7 * ((X.ml + Y.ml + 31) >> 5) + 30;
  if (mg_cost >= bs_cost) return false;
  uint32_t c = merge_count(X.m, X.ml, Y.m, Y.ml, label, A.lab, lane);
  if (X.xl) c += probe_count(X.x, X.xl, Y.m, Y.ml, label, A.lab, lane, vlo, vhi);
  if (Y.xl) c += probe_count(Y.x, Y.xl, X.m, X.ml, label, A.lab, lane, vlo, vhi);
  if (X.xl && Y.xl) c += probe_count(X.x, X.xl, Y.x, Y.xl, label, A.lab, lane, vlo, vhi);
  for (int e = 0; e < nexcl; ++e) {
    const int32_t v = excl[e];
    if (v > vlo && v < vhi && (label < 0 || A.lab[v] == (uint16_t)label) && contains(X, v) && contains(Y, v)) --c;
  }
  *out = c;
  return true;
}

// ---- run-shared bitmap count ------------------------------------------------------
// The run's x2 list P is hashed once into a per-warp shared bitmap; each entry then streams its other list X
// coalesced (32 consecutive elements per warp step, independent loads) and an element survives the bitmap
// test only if its hash bit is set — about (matches + |P|/bits) of them — and is then verified exactly by a
// binary search of P. Exact: every element of X ∩ P has its bit set; the bitmap only filters.
constexpr int kBmLog2 = GCSM_BM_INTS > 0 ? 5 + __builtin_ctz(GCSM_BM_INTS) : 5;
__device__ __forceinline__ uint32_t bm_hash(int32_t v) { return ((uint32_t)v * 2654435761u) >> (32 - kBmLog2); }

__device__ __forceinline__ void bm_build(uint32_t *bm, const int32_t *P, uint32_t n, int lane) {
  __syncwarp();
  for (uint32_t i = lane; i < (uint32_t)GCSM_BM_INTS; i += 32) bm[i] = 0;
  __syncwarp();
  for (uint32_t i = lane; i < n; i += 32) {
    const uint32_t h = bm_hash(P[i]);
    atomicOr(&bm[h >> 5], 1u << (h & 31));
  }
  __syncwarp();
}

__device__ __forceinline__ uint32_t bm_count(const MatchArgs &A, const uint32_t *bm, const LRef &X, const LRef &P,
                                             const int32_t *excl, int nexcl, int label, int lane, int32_t vlo,
                                             int32_t vhi) {
  uint32_t cnt = 0;
  auto visit = [&](const int32_t *seg, uint32_t n) {
    for (uint32_t i = lane; i < n; i += 32) {
      const int32_t v = seg[i];
      if (v <= vlo || v >= vhi) continue;
      const uint32_t h = bm_hash(v);
      bool in = false;
      if ((bm[h >> 5] >> (h & 31)) & 1u) in = bsearch_has(P.m, P.ml, v);
      if (!in && P.xl) in = bsearch_has(P.x, P.xl, v);
      if (!in) continue;
      if (label >= 0 && A.lab[v] != (uint16_t)label) continue;
      bool ex = false;
      for (int e = 0; e < nexcl; ++e) ex |= v == excl[e];
      cnt += !ex;
    }
  };
  visit(X.m, X.ml);
  if (X.xl) visit(X.x, X.xl);
#pragma unroll
  for (int o = 16; o; o >>= 1) cnt += __shfl_xor_sync(kFull, cnt, o);
  return cnt;
}

// Symmetry-breaking range of position p: vlo < candidate < vhi (counts scale by |Aut_L|).
__device__ __forceinline__ void range_of(const LevelPlan &Lp, const int32_t *f, int32_t *vlo, int32_t *vhi) {
  int32_t lo = INT_MIN, hi = INT_MAX;
  for (int i = 0; i < Lp.nlo; ++i) lo = max(lo, f[Lp.lo[i]]);
  for (int i = 0; i < Lp.nhi; ++i) hi = min(hi, f[Lp.hi[i]]);
  *vlo = lo;
  *vhi = hi;
}

__device__ __forceinline__ uint32_t lower_idx(const int32_t *a, uint32_t n, int32_t v) {
  uint32_t lo = 0, hi = n;
  while (lo < hi) {
    const uint32_t mid = (lo + hi) >> 1;
    if (a[mid] < v) lo = mid + 1;
    else hi = mid;
  }
  return lo;
}

// Narrow the device-resident main runs to the range (vlo, vhi): the sorted lists lose the elements no
// candidate may take, so every intersection below reads fewer of them.
__device__ __forceinline__ void trim_lists(LRef *L, int nl, int32_t vlo, int32_t vhi) {
  if (vlo == INT_MIN && vhi == INT_MAX) return;
  for (int p = 0; p < nl; ++p) {
    if (!L[p].dev || L[p].ml == 0) continue;
    const uint32_t b = vlo == INT_MIN ? 0 : lower_idx(L[p].m, L[p].ml, vlo + 1);
    const uint32_t e = vhi == INT_MAX ? L[p].ml : lower_idx(L[p].m, L[p].ml, vhi);
    L[p].m += b;
    L[p].ml = e > b ? e - b : 0;
  }
}

// Lists of position p for the current partial match f (positions 0..p-1).
// Returns the number of probe lists written to L and sets *drv (index of the
// smallest list) or uses the reused set.
__device__ __forceinline__ int gather_lists(const MatchArgs &A, const LevelPlan &Lp, const int32_t *f, LRef *L,
                                            int *drv, Acc &acc, int lane, const Pinned &pin = Pinned()) {
  int nl = 0;
  uint32_t best = 0xffffffffu;
  *drv = 0;
  if (Lp.reuse >= 0) {
    for (int r = 0; r < Lp.nrest; ++r) {
      const int b = Lp.rest[r];
      L[nl++] = list_of(A, f[Lp.bpos[b]], Lp.bview[b], acc, lane, pin);
    }
    return nl;
  }
  for (int b = 0; b < Lp.nb; ++b) {
    L[nl] = list_of(A, f[Lp.bpos[b]], Lp.bview[b], acc, lane, pin);
    const uint32_t sz = L[nl].ml + L[nl].xl;
    if (sz < best) {
      best = sz;
      *drv = nl;
    }
    ++nl;
  }
  return nl;
}

__device__ __forceinline__ void emit_tuples(const MatchArgs &A, const DevPlan &P, const int32_t *f, int kind,
                                            const int32_t *cand, uint32_t c, int lane) {
  unsigned long long base = 0;
  if (lane == 0) base = atomicAdd(&A.cnt[kind ? CNT_TUP_REM : CNT_TUP_ADD], (unsigned long long)c);
  base = __shfl_sync(kFull, base, 0);
  int32_t *T = kind ? A.tup_rem : A.tup_add;
  const uint64_t cap = kind ? A.tup_rem_cap : A.tup_add_cap;
  const int k = A.k;
  for (uint32_t i = lane; i < c; i += 32) {
    if (base + i >= cap) break;
    int32_t *t = T + (base + i) * (uint64_t)k;
    for (int p = 0; p < k - 1; ++p) t[P.order[p]] = f[p];
    t[P.order[k - 1]] = cand[i];
  }
}

__device__ __forceinline__ void flush(const MatchArgs &A, const Acc &acc, int lane) {
  __syncwarp();
  if (lane == 0) {
    if (acc.add) atomicAdd(&A.cnt[CNT_ADDED], acc.add);
    if (acc.rem) atomicAdd(&A.cnt[CNT_REMOVED], acc.rem);
    const int dst[kSN] = {A.acc_base + 0, A.acc_base + 1, A.acc_base + 2, CNT_COPIED, CNT_STAGE_FILL,
                          CNT_STAGE_LISTS, CNT_STAGE_HIT, CNT_PEER};
#pragma unroll
    for (int i = 0; i < kSN; ++i)
      if (acc.s[i]) atomicAdd(&A.cnt[dst[i]], acc.s[i]);
  }
}

// Level 2 (BFS step): warp per unit.
template <bool LIST>
__global__ void __launch_bounds__(kBlock, 4) k_level2(const __grid_constant__ MatchArgs A) {
  const int lane = threadIdx.x & 31;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  int32_t *buf = A.scratch + gw * A.scratch_stride;
  int32_t *gstage = buf + A.scratch_stride - 2 * (int64_t)A.dcap;
  extern __shared__ int4 smem_raw[];
  int32_t *sm = reinterpret_cast<int32_t *>(smem_raw) + (threadIdx.x >> 5) * kSmemInts;
  __shared__ unsigned long long s_stats[kWarps][kSN];
  Acc acc;
  acc.init(s_stats[threadIdx.x >> 5], lane);
  for (;;) {
    unsigned long long u = 0;
    if (lane == 0) u = atomicAdd(&A.cnt[CNT_CURSOR0], 1ull);
    u = __shfl_sync(kFull, u, 0);
    if ((int64_t)u >= A.n_units) break;
    const Unit U = A.units[u];
    const DevPlan &P = A.plans[U.plan];
    const int32_t f[2] = {U.a, U.b};
    if (A.k == 2) {  // single-edge query: the seed itself is the embedding
      if (P.kind) acc.rem += 1;
      else acc.add += 1;
      if (LIST) {
        if (lane == 0) {
          const unsigned long long base = atomicAdd(&A.cnt[P.kind ? CNT_TUP_REM : CNT_TUP_ADD], 1ull);
          int32_t *T = P.kind ? A.tup_rem : A.tup_add;
          if (base < (P.kind ? A.tup_rem_cap : A.tup_add_cap)) {
            T[base * 2 + P.order[0]] = U.a;
            T[base * 2 + P.order[1]] = U.b;
          }
        }
      }
      continue;
    }
    const LevelPlan &L2 = P.lv[2];
    LRef L[7];
    int drv;
    const int nl = gather_lists(A, L2, f, L, &drv, acc, lane);
    stage_lists(A, L, nl, drv, false, 0, sm, kSmemInts, gstage, lane, acc);
    int32_t vlo, vhi;
    range_of(L2, f, &vlo, &vhi);
    trim_lists(L, nl, vlo, vhi);
    int32_t excl[2];
    int nex = 0;
    for (int i = 0; i < L2.ninj; ++i) excl[nex++] = f[L2.inj[i]];
    if (A.k == 3 && !LIST) {
      uint32_t c;
      if (nl != 2 || !count2(A, L, drv, excl, nex, L2.label, lane, &c, vlo, vhi))
        c = warp_isect<false>(A, nullptr, 0, L, nl, drv, excl, nex, L2.label, nullptr, lane, vlo, vhi);
      if (P.kind) acc.rem += c;
      else acc.add += c;
      continue;
    }
    const uint32_t c = warp_isect<true>(A, nullptr, 0, L, nl, drv, excl, nex, L2.label, buf, lane, vlo, vhi);
    __syncwarp();
    if (A.k == 3) {  // LIST
      if (P.kind) acc.rem += c;
      else acc.add += c;
      emit_tuples(A, P, f, P.kind, buf, c, lane);
      __syncwarp();
      continue;
    }
    unsigned long long off = 0;
    if (lane == 0 && c) off = atomicAdd(&A.cnt[CNT_F2], (unsigned long long)c);
    off = __shfl_sync(kFull, off, 0);
    if (off + c > (unsigned long long)A.f2_cap) {
      if (lane == 0) atomicOr(&A.cnt[CNT_OVERFLOW], 1ull);
      continue;
    }
    int32_t *f2c = reinterpret_cast<int32_t *>(A.f2);
    int32_t *f2u = f2c + A.f2_cap;
    for (uint32_t i = lane; i < c; i += 32) {
      f2c[off + i] = buf[i];
      f2u[off + i] = (int32_t)u;
    }
    if (lane == 0) A.useg[u] = make_int2((int)off, (int)c);
    __syncwarp();
  }
  flush(A, acc, lane);
}

__device__ __forceinline__ unsigned long long warp_sum64(unsigned long long x) {
#pragma unroll
  for (int o = 16; o; o >>= 1) x += __shfl_xor_sync(kFull, x, o);
  return x;
}

// Do the sorted runs a[0..na) and b[0..nb) share an element? Merge path over the warp (co-rank split, each lane
// merges its diagonal range): O((na + nb) / 32) steps, for two long device-resident runs whose lane-parallel
// binary-search test would take min(na, nb) / 32 rounds of log2 steps (the level-3 filter of a C4 hub node).
__device__ __forceinline__ bool merge_meet(const int32_t *a, uint32_t na, const int32_t *b, uint32_t nb, int lane) {
  const uint32_t T = na + nb;
  const uint32_t d0 = (uint32_t)(((uint64_t)T * (uint32_t)lane) >> 5);
  const uint32_t d1 = (uint32_t)(((uint64_t)T * (uint32_t)(lane + 1)) >> 5);
  uint32_t lo = d0 > nb ? d0 - nb : 0, hi = d0 < na ? d0 : na;
  while (lo < hi) {
    const uint32_t i = (lo + hi) >> 1;
    if (a[i] <= b[d0 - i - 1]) lo = i + 1;
    else hi = i;
  }
  uint32_t i = lo, j = d0 - lo;
  bool hit = false;
  // one step past the range as well: an equal pair split across two lanes' ranges is seen by the earlier lane
  while (i + j <= d1 && !hit) {
    const int32_t ai = i < na ? a[i] : INT_MAX;
    const int32_t bj = j < nb ? b[j] : INT_MAX;
    if (ai == bj && ai != INT_MAX) hit = true;
    i += ai <= bj;
    j += ai >= bj;
  }
  return __any_sync(kFull, hit);
}

// Level-3 filter (LevelPlan::fmask): position 4's candidates for a level-3 node x3 lie in
// F ∩ view(N(x3)), where F = F[0..nF1) ∪ F2[0..nF-nF1) (two sorted runs, label-filtered) is the intersection of position 4's lists fixed for the whole
// level-2 entry. Lane i tests node i: does its own list meet F? Nodes that cannot (almost all of them on C4) are
// dropped from the level-3 set before the warp-wide DFS visits them; the test ignores injectivity and symmetry
// ranges, so it only ever keeps too much (exact). Survivors go to out (may be set3 itself: compaction in place);
// returns their number.
// The byte counters go out through facc[6] (hit, miss, delta, staged, peer, filled) and fl[1] (lists filled): the
// warp's shared DFS record, so that the caller's Acc is never address-taken.
__device__ __noinline__ uint32_t filter_level3(const MatchArgs &A, int vw, const int32_t *set3, uint32_t n3,
                                               int32_t *out, const int32_t *F, const int32_t *F2, uint32_t nF1,
                                               uint32_t nF, unsigned long long *stats, int lane) {
  Acc acc;  // statistics only: the caller's warp block
  acc.s = stats;
  acc.l0 = lane == 0;
  uint32_t w = 0;
  unsigned long long hb = 0, mb = 0, db = 0, sb = 0, pb = 0;  // per-lane algorithmic bytes: hit, miss, delta, staged, peer
  for (uint32_t base = 0; base < n3; base += 32) {
    const uint32_t i = base + lane;
    const bool act = i < n3;
    const int32_t v = act ? set3[i] : 0;
    const int32_t *m = nullptr, *x = nullptr;
    uint32_t ml = 0, xl = 0;
    bool need = false;
    if (act) {
      const int4 raw = __ldg(reinterpret_cast<const int4 *>(A.vdesc + v));
      m = reinterpret_cast<const int32_t *>((unsigned long long)(unsigned)raw.x |
                                            ((unsigned long long)(unsigned)raw.y << 32));
      ml = (uint32_t)raw.z;
      const uint32_t upd = (uint32_t)raw.w;
      if (upd != 0 && vw != VIEW_S) {
        const int4 e = __ldg(reinterpret_cast<const int4 *>(A.drec + (upd - 1)));
        x = A.dlist + (vw == VIEW_NEW ? e.x : e.z);
        xl = (uint32_t)(vw == VIEW_NEW ? e.y : e.w);
      }
      mark_touched(A, v);
      db += 4ull * xl;
      const char *pc = reinterpret_cast<const char *>(m);
      if (pc >= A.cache_lo && pc < A.cache_hi) {
        hb += 4ull * ml;
      } else if (pc >= A.ubuf_lo && pc < A.ubuf_hi) {
        db += 4ull * ml;
      } else {
        mb += 4ull * ml;
        const int32_t *q = (A.npeer && upd == 0 && ml > 0) ? peer_lookup(A, v, ml) : nullptr;
        if (q) {
          m = q;
          pb += 4ull * ml;
        } else if (A.stage_state && ml >= A.stage_min) {
          const unsigned long long st = stage_word(A.stage_state + v);
          if ((st >> 40) == A.stage_epoch && (st & kStReady) && (st & kStOff) != kStOff) {
            m = A.stage_arena + (st & kStOff);
            sb += 4ull * ml;
          } else {
            need = true;
          }
        }
      }
    }
    // lists not staged yet: the warp fetches them once (every later reader in the batch finds them in HBM)
    for (unsigned nm = __ballot_sync(kFull, need); nm; nm &= nm - 1) {
      const int l = __ffs(nm) - 1;
      const int32_t vl = __shfl_sync(kFull, v, l);
      const unsigned long long hp = __shfl_sync(kFull, (unsigned long long)m, l);
      const uint32_t mll = __shfl_sync(kFull, ml, l);
      const int32_t *q = stage_resolve(A, vl, reinterpret_cast<const int32_t *>(hp), mll, acc, lane);
      if (lane == l) m = q;
    }
    bool hit = false;
    const uint32_t nF2 = nF - nF1;
    // a node whose test streams more than kFiltLane elements is tested by the whole warp below (one lane alone took
    // up to 20 ms on a C4 hub node: profiles/c4_trace_r02_v7.txt)
    const bool big = act && min(ml + xl, nF) > kFiltLane;
    if (act && !big) {
      if (ml + xl <= nF) {  // stream the node's list, probe F (its two sorted runs)
        for (uint32_t j = 0; j < ml && !hit; ++j) hit = bsearch_has(F, nF1, m[j]) || (nF2 && bsearch_has(F2, nF2, m[j]));
        for (uint32_t j = 0; j < xl && !hit; ++j) hit = bsearch_has(F, nF1, x[j]) || (nF2 && bsearch_has(F2, nF2, x[j]));
      } else {  // stream F, probe the node's list
        for (uint32_t j = 0; j < nF && !hit; ++j) {
          const int32_t fj = j < nF1 ? F[j] : F2[j - nF1];
          hit = bsearch_has(m, ml, fj) || (xl && bsearch_has(x, xl, fj));
        }
      }
    }
    for (unsigned bgm = __ballot_sync(kFull, big); bgm; bgm &= bgm - 1) {  // warp-wide tests, early exit on a hit
      const int l = __ffs(bgm) - 1;
      const int32_t *bm_ = reinterpret_cast<const int32_t *>(__shfl_sync(kFull, (unsigned long long)m, l));
      const int32_t *bx = reinterpret_cast<const int32_t *>(__shfl_sync(kFull, (unsigned long long)x, l));
      const uint32_t bml = __shfl_sync(kFull, ml, l), bxl = __shfl_sync(kFull, xl, l);
      bool found = false;
      const char *pc = reinterpret_cast<const char *>(bm_);
      const bool bdev = (pc >= A.cache_lo && pc < A.cache_hi) || (pc >= A.ubuf_lo && pc < A.ubuf_hi) ||
                        (A.stage_arena && bm_ >= A.stage_arena && bm_ < A.stage_arena + A.stage_cap) ||
                        (pc >= reinterpret_cast<const char *>(A.scratch) &&
                         pc < reinterpret_cast<const char *>(A.scratch_end)) || __isShared(bm_);
      if (bdev && nF1 && bml && (uint64_t)nF1 + bml < 8ull * min(nF1, bml)) {
        // two long runs: merge path for main x main, lane-parallel probes for the short delta runs
        found = merge_meet(F, nF1, bm_, bml, lane);
        for (uint32_t j0 = 0; j0 < bxl && !found; j0 += 32) {
          const uint32_t j = j0 + lane;
          const bool h = j < bxl && (bsearch_has(F, nF1, bx[j]) || (nF2 && bsearch_has(F2, nF2, bx[j])));
          found = __any_sync(kFull, h);
        }
        for (uint32_t j0 = 0; j0 < nF2 && !found; j0 += 32) {
          const uint32_t j = j0 + lane;
          const bool h = j < nF2 && bsearch_has(bm_, bml, F2[j]);
          found = __any_sync(kFull, h);
        }
      } else if (bml + bxl <= nF) {
        for (uint32_t j0 = 0; j0 < bml + bxl && !found; j0 += 32) {
          const uint32_t j = j0 + lane;
          bool h = false;
          if (j < bml + bxl) {
            const int32_t u = j < bml ? bm_[j] : bx[j - bml];
            h = bsearch_has(F, nF1, u) || (nF2 && bsearch_has(F2, nF2, u));
          }
          found = __any_sync(kFull, h);
        }
      } else {
        for (uint32_t j0 = 0; j0 < nF && !found; j0 += 32) {
          const uint32_t j = j0 + lane;
          bool h = false;
          if (j < nF) {
            const int32_t fj = j < nF1 ? F[j] : F2[j - nF1];
            h = bsearch_has(bm_, bml, fj) || (bxl && bsearch_has(bx, bxl, fj));
          }
          found = __any_sync(kFull, h);
        }
      }
      if (lane == l) hit = found;
    }
    const unsigned hm = __ballot_sync(kFull, hit);
    if (hit) out[w + __popc(hm & ((1u << lane) - 1u))] = v;
    w += __popc(hm);
    __syncwarp();
  }
  acc.stat(kSHit, warp_sum64(hb));
  acc.stat(kSMiss, warp_sum64(mb));
  acc.stat(kSDelta, warp_sum64(db));
  acc.stat(kSSHit, warp_sum64(sb));
  acc.stat(kSPeer, warp_sum64(pb));
  __syncwarp();
  return w;
}

// Warp-uniform DFS state of k_extend in shared memory (every lane writes the same values): the partial match, the
// candidate sets and iterators per level and the list descriptors of the current intersection. Indexed at run time
// (the query size and plans are runtime data), these arrays lived in local memory and their spills dominated the
// kernel's DRAM traffic (profiles/ncu_c4_r02_v2.md: 48 GB per prism6 launch for ~1 GB of lists).
struct WarpDfs {
  int32_t f[GCSM_MAXK];
  const int32_t *set[GCSM_MAXK];
  uint32_t sz[GCSM_MAXK], it[GCSM_MAXK];
  LRef L[7], Lx[7];
  int32_t excl[GCSM_MAXK];
  unsigned long long stats[kSN];  // this warp's byte statistics (Acc)
};
constexpr int kExtSmemBytes = kSmemBytes + kWarps * (int)sizeof(WarpDfs);

// Levels 3..k-1 (DFS): warp per level-2 frontier entry.
template <bool LIST, int KK>  // KK: compile-time query size (4: the level-3 count only), 0 = any
__global__ void __launch_bounds__(kBlock, GCSM_MINBLOCKS) k_extend(const __grid_constant__ MatchArgs A) {
  const int lane = threadIdx.x & 31;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  int32_t *stack = A.scratch + gw * A.scratch_stride;  // buffer for position p: stack + (p - 3) * dcap
  int32_t *gstage = stack + A.scratch_stride - 2 * (int64_t)A.dcap;
  int32_t *pstage = gstage - (int64_t)A.dcap;  // persistent copy of the current x2's main list
  extern __shared__ int4 smem_raw[];
  uint32_t *bm = reinterpret_cast<uint32_t *>(smem_raw) + (threadIdx.x >> 5) * kSmemInts;
  int32_t *sm = reinterpret_cast<int32_t *>(bm) + GCSM_BM_INTS;  // pin area, then transient staging
  constexpr uint32_t kSlice = kSmemInts - GCSM_BM_INTS;
  WarpDfs &Wd = *reinterpret_cast<WarpDfs *>(reinterpret_cast<char *>(smem_raw) + kSmemBytes +
                                             (threadIdx.x >> 5) * sizeof(WarpDfs));
  int32_t *const f = Wd.f;
  const int32_t **const set = Wd.set;
  uint32_t *const sz = Wd.sz, *const it = Wd.it;
  const int k = KK ? KK : A.k;
  int32_t *lastbuf = stack + (int64_t)(k > 4 ? k - 4 : 0) * A.dcap;  // LIST: last-level candidates
  int32_t *hbuf = stack + (int64_t)((k > 4 ? k - 4 : 0) + (LIST ? 1 : 0)) * A.dcap;  // hoisted last-level set
  int32_t *fbuf = hbuf + A.dcap;                                                        // level-3 filter set F
  int32_t *ibuf = fbuf + A.dcap;                                 // level-3 iteration list (filtered, set reused)
  const int64_t n_f2 = (int64_t)*(volatile unsigned long long *)&A.cnt[CNT_F2];
  const int32_t *f2c = reinterpret_cast<const int32_t *>(A.f2);
  const int32_t *f2u = f2c + A.f2_cap;
  // work grab size: runs of up to kChunk entries, smaller when the frontier would leave warps idle
  const int64_t warps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const int64_t chunk = max((int64_t)1, min((int64_t)kChunk, n_f2 / (4 * warps)));
  Acc acc;
  acc.init(Wd.stats, lane);
  Pinned pin;
  unsigned long long x_entries = 0, x_pruned = 0, x_l3 = 0, x_l4 = 0, x_last = 0, x_l3f = 0;  // work profile
  uint32_t pin_sm = 0;  // ints of the shared slice held by the pinned x2 list
  int64_t ci = 0, c_end = 0, c_start = 0;
  bool producing = true;  // phase 1: walk the (grouped) frontier; phase 2 (k >= 5): take shared level-3 tasks
  const bool sharing = KK == 0 && !LIST && k >= 5 && A.tasks != nullptr;
  const long long t_start = clock64();
  long long t_ph1 = 0, t_entry = 0, t_emax = 0;  // timing profile (CNT_XT)
  long long tp[5] = {0, 0, 0, 0, 0}, tpm[5] = {0, 0, 0, 0, 0};  // this entry's phases / the warp's maxima:
                                                                  // hoist, F, level-3 set, filter, rest
  for (;;) {
    int64_t e;
    bool task = false;
    Task tk;
    if (producing) {
      if (ci >= c_end) {  // grab the next chunk of the (x2-grouped) frontier order
        unsigned long long c0 = 0;
        if (lane == 0) c0 = atomicAdd(&A.cnt[CNT_CURSOR1], (unsigned long long)chunk);
        c0 = __shfl_sync(kFull, c0, 0);
        if (sharing && c_end > 0 && lane == 0) {  // the previous chunk is finished (tasks published)
          __threadfence();
          atomicAdd(&A.cnt[CNT_PRODUCERS], (unsigned long long)(c_end - c_start));
        }
        if ((int64_t)c0 >= n_f2) {
          t_ph1 = clock64() - t_start;
          if (!sharing) break;
          producing = false;
          pin.v = -1;
          pin.bm_v = -1;
          pin_sm = 0;
          continue;
        }
        c_start = (int64_t)c0;
        ci = (int64_t)c0;
        c_end = min((int64_t)c0 + chunk, n_f2);
        pin.v = -1;
        pin.bm_v = -1;
        pin_sm = 0;
      }
      e = A.group ? A.group[ci] : ci;
      const int32_t x2 = f2c[e];
      if (x2 != pin.v) {
        // run of entries sharing x2 in this chunk: stage x2's zero-copy main list once for all of them
        int64_t j = ci + 1 + lane;
        const bool same = j < c_end && f2c[A.group ? A.group[j] : j] == x2;
        const unsigned run_mask = __ballot_sync(kFull, same);
        const int run = 1 + (run_mask == kFull ? 32 : __ffs(~run_mask) - 1);  // entries of this run (capped at 33)
        pin.v = -1;
        const int4 raw = __ldg(reinterpret_cast<const int4 *>(A.vdesc + x2));
        pin.rv = x2;
        pin.raw = raw;
        const int32_t *mp = reinterpret_cast<const int32_t *>((unsigned long long)(unsigned)raw.x |
                                                                ((unsigned long long)(unsigned)raw.y << 32));
        const uint32_t ml = (uint32_t)raw.z;
        bool miss = !is_hit(A, mp), staged = false;
        if (lane == 0) mark_touched(A, x2);
        if (miss && A.npeer && raw.w == 0 && ml > 0) {  // a linked peer's HBM cache holds it
          const int32_t *q = peer_lookup(A, x2, ml);
          if (q) {
            mp = q;
            miss = false;
            staged = true;  // device-resident: served in place for the run unless pinned in shared memory
          }
        }
        if (miss && A.stage_state && ml >= A.stage_min) {  // the run's x2 list, fetched once per batch
          const int32_t *sp = stage_resolve(A, x2, mp, ml, acc, lane);
          if (sp != mp) {
            mp = sp;
            miss = false;
            staged = true;
          }
        }
        const uint32_t ml4 = (ml + 3) & ~3u;
        pin_sm = 0;
        pin.bm_v = -1;
        if (run >= 2 && ml >= 32 && ml4 <= GCSM_PIN_SMEM_MAX) {  // fits the shared slice: pin hits and misses
          warp_copy(sm, mp, ml, lane);
          if (miss) acc.stat(kSCopied, 4ull * ml);
          __syncwarp();
          pin.v = x2;
          pin.p = sm;
          pin_sm = ml4;
        } else if (run >= 2 && ml >= 32 && miss && ml <= (uint32_t)A.dcap) {
          warp_copy(pstage, mp, ml, lane);
          acc.stat(kSCopied, 4ull * ml);
          __syncwarp();
          pin.v = x2;
          pin.p = pstage;
        }
        if (staged && pin.v != x2) {  // served in place from the batch arena (HBM) for the whole run
          pin.v = x2;
          pin.p = mp;
        }
        if (GCSM_BM_INTS > 0 && run >= 2 && ml >= 32 && (pin.v == x2 || !miss)) {
          bm_build(bm, pin.v == x2 ? pin.p : mp, ml, lane);
          pin.bm_v = x2;
        }
      }
      ++ci;
    } else {
      // phase 2: take a ticket (unique task index); wait until that task is published, or leave when every
      // frontier entry has been walked (the task tail is final) and the ticket lies past it
      unsigned long long h = 0;
      if (lane == 0) h = atomicAdd(&A.cnt[CNT_HEAD], 1ull);
      h = __shfl_sync(kFull, h, 0);
      int state = 0;  // 1: task h is ready, 2: no such task will exist
      if (lane == 0) {
        unsigned ns = 64;
        for (;;) {
          const unsigned long long tail = *(volatile unsigned long long *)&A.cnt[CNT_TAIL];
          if (h < tail) {
            if (h >= A.task_cap) { state = 3; break; }  // reserved past the array: its owner kept the work
            if (*(volatile int32_t *)&A.task_ready[h] == A.task_gen) { state = 1; break; }
          } else {
            const unsigned long long done = *(volatile unsigned long long *)&A.cnt[CNT_PRODUCERS];
            __threadfence();  // the producers fence between publishing and counting an entry as walked
            if ((int64_t)done >= n_f2 && h >= *(volatile unsigned long long *)&A.cnt[CNT_TAIL]) { state = 2; break; }
          }
          __nanosleep(ns);
          if (ns < 4096) ns <<= 1;
        }
      }
      state = __shfl_sync(kFull, state, 0);
      if (state == 2) break;
      if (state == 3) continue;
      __syncwarp();
      __threadfence();
      // other SMs wrote the task and its arena slice during this launch: read them through L2 (ld.global.cg),
      // never from a possibly stale L1 line
      {
        const unsigned long long *src = reinterpret_cast<const unsigned long long *>(&A.tasks[h]);
        unsigned long long w[7];
#pragma unroll
        for (int i = 0; i < 7; ++i) w[i] = __ldcg(src + i);
        memcpy(&tk, w, sizeof(Task));
      }
      if (tk.lo >= tk.hi) continue;  // an empty placeholder (its producer kept the work)
      e = tk.e;
      task = true;
    }
    {
      const long long now = clock64();
      if (t_entry) {
        t_emax = max(t_emax, now - t_entry);
        long long rest = now - t_entry;
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          tpm[i] = max(tpm[i], tp[i]);
          rest -= tp[i];
        }
        tpm[4] = max(tpm[4], rest);
      }
#pragma unroll
      for (int i = 0; i < 4; ++i) tp[i] = 0;
      t_entry = now;
    }
    const int32_t ui = f2u[e];
    const Unit U = A.units[ui];
    const DevPlan &P = A.plans[U.plan];
    const int2 seg = A.useg[ui];
    if (!task) ++x_entries;
    __syncwarp();  // every lane is done with the previous entry's state
    f[0] = U.a;
    f[1] = U.b;
    f[2] = f2c[e];
    set[2] = f2c + seg.x;
    sz[2] = (uint32_t)seg.y;
    uint32_t end3 = 0xffffffffu;  // level-3 iteration bound (a task's slice)
    int lvl = 2;   // deepest position with a chosen element
    bool descend = true;
    // hoisted last-level set (LevelPlan::hmask): ∩ of the last position's lists fixed at level 2, label-filtered
    const int32_t *hset = nullptr;
    uint32_t hn = 0;
    if (task && tk.xoff != ~0ull) {  // H and F as the producer computed them (L2 reads: written in this launch)
      hn = tk.hn;
      for (uint32_t i = lane; i < hn; i += 32) hbuf[i] = __ldcg(A.arena + tk.xoff + i);
      for (uint32_t i = lane; i < tk.nF; i += 32) fbuf[i] = __ldcg(A.arena + tk.xoff + hn + i);
      __syncwarp();
      if (KK == 0 && P.lv[k - 1].hmask && A.hoist) hset = hbuf;
    } else if (KK == 0 && P.lv[k - 1].hmask && A.hoist) {
      const LevelPlan &Lh = P.lv[k - 1];
      LRef *const Lx = Wd.Lx;
      int nx = 0, hdrv = 0;
      uint32_t best = 0xffffffffu;
      for (int b = 0; b < Lh.nb; ++b)
        if ((Lh.hmask >> b) & 1) {
          Lx[nx] = list_of(A, f[Lh.bpos[b]], Lh.bview[b], acc, lane, pin);
          const uint32_t szx = Lx[nx].ml + Lx[nx].xl;
          if (szx < best) {
            best = szx;
            hdrv = nx;
          }
          ++nx;
        }
      if (nx == 1 && Lh.label < 0 && Lx[0].dev && Lx[0].xl == 0) {  // one device-resident run: referenced
        hset = Lx[0].m;
        hn = Lx[0].ml;
      } else {
        const long long t0 = clock64();
        hn = warp_isect<true>(A, nullptr, 0, Lx, nx, hdrv, nullptr, 0, Lh.label, hbuf, lane);
        __syncwarp();
        hset = hbuf;
        tp[0] += clock64() - t0;
      }
      if (hn == 0) {  // no candidate for the last position anywhere below this entry
        ++x_pruned;
        continue;
      }
    }
    // level-3 filter set F (LevelPlan::fmask): ∩ of position 4's lists fixed for this entry, label-filtered
    uint32_t nF = 0, nF1 = 0;  // F = fset[0..nF1) ∪ fset2[0..nF-nF1), two sorted runs
    const int32_t *fset = fbuf, *fset2 = fbuf;
    const bool filt = KK == 0 && k >= 5 && P.lv[4].fmask != 0 && A.filter3;
    if (filt && task && tk.xoff != ~0ull) {
      nF1 = tk.nF1;
      nF = tk.nF;
      fset2 = fbuf + nF1;
    } else if (filt) {
      const LevelPlan &L4 = P.lv[4];
      LRef *const Lx = Wd.Lx;
      int nx = 0, fdrv = 0;
      uint32_t best = 0xffffffffu;
      for (int b = 0; b < L4.nb; ++b)
        if ((L4.fmask >> b) & 1) {
          Lx[nx] = list_of(A, f[L4.bpos[b]], L4.bview[b], acc, lane, pin);
          const uint32_t szx = Lx[nx].ml + Lx[nx].xl;
          if (szx < best) {
            best = szx;
            fdrv = nx;
          }
          ++nx;
        }
      // F as two sorted runs: survivors of the driver's main run, then of its delta run (an updated vertex's
      // view is main ∪ delta, each sorted, not sorted together); the filter binary-searches each run
      const LRef dfull = Lx[fdrv];
      if (nx == 1 && L4.label < 0 && dfull.dev) {  // F is one device-resident view: referenced, not copied
        fset = dfull.m;
        nF1 = dfull.ml;
        fset2 = dfull.x;
        nF = dfull.ml + dfull.xl;
      } else {
      Lx[fdrv].xl = 0;
      const long long t0 = clock64();
      nF1 = warp_isect<true>(A, nullptr, 0, Lx, nx, fdrv, nullptr, 0, L4.label, fbuf, lane);
      __syncwarp();
      nF = nF1;
      fset2 = fbuf + nF1;
      if (dfull.xl) {
        Lx[fdrv].m = dfull.x;
        Lx[fdrv].ml = dfull.xl;
        Lx[fdrv].dev = true;
        nF += warp_isect<true>(A, nullptr, 0, Lx, nx, fdrv, nullptr, 0, L4.label, fbuf + nF1, lane);
        __syncwarp();
      }
      tp[1] += clock64() - t0;
      }
      if (nF == 0) {  // no position-4 candidate for any level-3 node of this entry
        ++x_pruned;
        continue;
      }
    }
    // level 3 is iterated over it3p[0..it3n): position 3's set itself, or — when the level-3 filter ran and a later
    // position reuses position 3's whole set (code motion) — the filter's survivors in their own buffer
    const int32_t *it3p = nullptr;
    uint32_t it3n = 0;
    bool reuse3 = false;
    for (int q = 4; q < k; ++q) reuse3 |= P.lv[q].reuse == 3;
    if (task && tk.pad == kTaskFilter) {
      // an unfiltered slice: copy it (or the whole set when a later position reuses it), filter it here
      int32_t *own = stack;
      const uint32_t lo = reuse3 ? 0 : tk.lo, cnt = reuse3 ? tk.n : tk.hi - tk.lo;
      for (uint32_t i = lane; i < cnt; i += 32) own[i] = __ldcg(A.arena + tk.off + lo + i);
      __syncwarp();
      const int32_t *slice = reuse3 ? own + tk.lo : own;
      const long long tf = clock64();
      it3n = filter_level3(A, P.lv[4].bview[P.lv[4].f3], slice, tk.hi - tk.lo, ibuf, fset, fset2, nF1, nF, acc.s, lane);
      tp[3] += clock64() - tf;
      x_l3f += it3n;
      it3p = ibuf;
      __syncwarp();
      set[3] = own;
      sz[3] = cnt;
      it[3] = 0;
      end3 = it3n;
      lvl = 3;
      descend = false;
    } else if (task) {
      int32_t *own = stack;  // this warp's level-3 buffer: a private, L1-safe copy of the shared set
      for (uint32_t i = lane; i < tk.n; i += 32) own[i] = __ldcg(A.arena + tk.off + i);
      it3p = own;
      it3n = tk.n;
      if (tk.pad) {  // the producer's filtered iteration list follows the set in the arena
        it3n = tk.pad - 1;
        for (uint32_t i = lane; i < it3n; i += 32) ibuf[i] = __ldcg(A.arena + tk.off + tk.n + i);
        it3p = ibuf;
      }
      __syncwarp();
      set[3] = own;
      sz[3] = tk.n;
      it[3] = tk.lo;
      end3 = tk.hi;
      lvl = 3;
      descend = false;
    }
    for (;;) {
      if (descend) {
        const int p = lvl + 1;  // compute candidates of position p
        const LevelPlan &Lp = P.lv[p];
        LRef *const L = Wd.L;
        int drv = 0;
        int nl = (p == k - 1 && hset) ? 0 : gather_lists(A, Lp, f, L, &drv, acc, lane, pin);
        int32_t *const excl = Wd.excl;
        int nex = 0;
        for (int i = 0; i < Lp.ninj; ++i) excl[nex++] = f[Lp.inj[i]];
        const int32_t *dset = Lp.reuse >= 0 ? set[Lp.reuse] : nullptr;
        uint32_t dn = Lp.reuse >= 0 ? sz[Lp.reuse] : 0;
        if (p == k - 1 && hset) {  // hoisted set drives; probes = the lists not hoisted
          int w2 = 0;
          for (int b = 0; b < Lp.nb; ++b)
            if (!((Lp.hmask >> b) & 1)) L[w2++] = list_of(A, f[Lp.bpos[b]], Lp.bview[b], acc, lane, pin);
          nl = w2;
          dset = hset;
          dn = hn;
        }
        uint32_t c = 0;
        int32_t vlo, vhi;
        range_of(Lp, f, &vlo, &vhi);
        // last level, two lists, one of them the run's x2 list in the bitmap: stream the other one
        bool merged = false;
        if (GCSM_BM_INTS > 0 && !LIST && p == k - 1 && !dset && nl == 2 && pin.bm_v >= 0 && !task) {
          const int pi = f[Lp.bpos[0]] == pin.bm_v ? 0 : (f[Lp.bpos[1]] == pin.bm_v ? 1 : -1);
          if (pi >= 0) {
            const LRef &X = L[1 - pi];
            const uint32_t nx = X.ml + X.xl, np = L[pi].ml + L[pi].xl;
            const uint32_t bm_cost = 8 * ((nx + 31) >> 5) + 24;
            const uint32_t d = min(nx, np), big = max(nx, np);
            const uint32_t bs_cost = ((d + 31) >> 5) * (7 * ilog2(big) + 12);
            if (bm_cost <= bs_cost && X.dev) {
              c = bm_count(A, bm, X, L[pi], excl, nex, Lp.label, lane, vlo, vhi);
              merged = true;
            }
          }
        }
        if (!merged) stage_lists(A, L, nl, drv, dset != nullptr, dn, sm + pin_sm, kSlice - pin_sm, gstage, lane, acc);
        if (!merged) trim_lists(L, nl, vlo, vhi);
        if (merged) {
          if (P.kind) acc.rem += c;
          else acc.add += c;
          descend = false;
        } else if (p == k - 1) {
          x_last += dset ? dn : (nl ? L[drv].ml + L[drv].xl : 0);
          if (LIST) {
            c = warp_isect<true>(A, dset, dn, L, nl, drv, excl, nex, Lp.label, lastbuf, lane, vlo, vhi);
            __syncwarp();
            emit_tuples(A, P, f, P.kind, lastbuf, c, lane);
            __syncwarp();
          } else if (dset || nl != 2 || !count2(A, L, drv, excl, nex, Lp.label, lane, &c, vlo, vhi)) {
            c = warp_isect<false>(A, dset, dn, L, nl, drv, excl, nex, Lp.label, nullptr, lane, vlo, vhi);
          }
          if (P.kind) acc.rem += c;
          else acc.add += c;
          descend = false;
        } else {
          int32_t *out = stack + (int64_t)(p - 3) * A.dcap;
          const long long t3 = clock64();
          sz[p] = warp_isect<true>(A, dset, dn, L, nl, drv, excl, nex, Lp.label, out, lane, vlo, vhi);
          if (p == 3) tp[2] += clock64() - t3;
          if (p == 3) x_l3 += sz[p];
          else if (p == 4) x_l4 += sz[p];
          if (p == 3) {
            it3p = out;
            it3n = sz[3];
          }
          const bool unf = p == 3 && filt && sharing && A.fsplit && sz[3] > kFSplitMin;  // shared unfiltered
          if (p == 3 && filt && sz[3] && !unf) {  // keep only the level-3 nodes whose own list meets F
            __syncwarp();
            int32_t *dst = reuse3 ? ibuf : out;
            const long long tf = clock64();
            it3n = filter_level3(A, P.lv[4].bview[P.lv[4].f3], out, sz[3], dst, fset, fset2, nF1, nF, acc.s, lane);
            tp[3] += clock64() - tf;
            it3p = dst;
            if (!reuse3) sz[3] = it3n;
            x_l3f += it3n;
          }
          __syncwarp();
          set[p] = out;
          it[p] = 0;
          lvl = p;
          descend = false;
          if (p == 3 && sharing && (unf || it3n > kSplitMin)) {
            // share this level-3 set: copy it (and a separate iteration list) to the arena and publish slices of the
            // iteration list as tasks (unf: slices of the unfiltered set, each filtered by its taker)
            const bool sep = !unf && it3p != out;
            const uint32_t tsz = unf ? kFTaskSize : kTaskSize;
            const uint32_t n3 = sz[3], ni = it3n, nt = (ni + tsz - 1) / tsz;
            const uint32_t nH = hset ? hn : 0, nFx = filt ? nF : 0;  // the entry's H and F go with the set
            const unsigned long long need = (unsigned long long)n3 + (sep ? ni : 0) + nH + nFx;
            unsigned long long off = 0, t0 = 0;
            if (lane == 0) {
              off = atomicAdd(&A.cnt[CNT_ARENA], need);
              t0 = atomicAdd(&A.cnt[CNT_TAIL], (unsigned long long)nt);
            }
            off = __shfl_sync(kFull, off, 0);
            t0 = __shfl_sync(kFull, t0, 0);
            const unsigned long long xoff = off + n3 + (sep ? ni : 0);
            if (off + need <= A.arena_cap && t0 + nt <= A.task_cap) {
              for (uint32_t i = lane; i < n3; i += 32) A.arena[off + i] = out[i];
              if (sep)
                for (uint32_t i = lane; i < ni; i += 32) A.arena[off + n3 + i] = it3p[i];
              for (uint32_t i = lane; i < nH; i += 32) A.arena[xoff + i] = hset[i];
              for (uint32_t i = lane; i < nFx; i += 32) A.arena[xoff + nH + i] = i < nF1 ? fset[i] : fset2[i - nF1];
              for (uint32_t t = lane; t < nt; t += 32) {
                Task q;
                q.e = e;
                q.off = off;
                q.n = n3;
                q.lo = t * tsz;
                q.hi = min(ni, (t + 1) * tsz);
                q.pad = unf ? kTaskFilter : (sep ? ni + 1 : 0);
                q.xoff = xoff;
                q.hn = nH;
                q.nF1 = filt ? nF1 : 0;
                q.nF = nFx;
                q.pad2 = 0;
                A.tasks[t0 + t] = q;
              }
              __threadfence();
              __syncwarp();
              for (uint32_t t = lane; t < nt; t += 32) *(volatile int32_t *)&A.task_ready[t0 + t] = A.task_gen;
              if (lane == 0) atomicAdd(&A.cnt[CNT_SPLIT], 1ull);
              end3 = 0;  // all of it delegated
            } else {
              // no room: publish empty tasks for the reserved slots so takers do not wait forever
              for (uint32_t t = lane; t < nt; t += 32) {
                if (t0 + t < A.task_cap) {
                  Task q;
                  q.e = e;
                  q.off = 0;
                  q.n = 0;
                  q.lo = q.hi = 0;
                  q.pad = 0;
                  q.xoff = ~0ull;
                  q.hn = q.nF1 = q.nF = q.pad2 = 0;
                  A.tasks[t0 + t] = q;
                }
              }
              __threadfence();
              __syncwarp();
              for (uint32_t t = lane; t < nt; t += 32)
                if (t0 + t < A.task_cap) *(volatile int32_t *)&A.task_ready[t0 + t] = A.task_gen;
            }
          }
        }
      }
      // choose the next element at the deepest open position (>= 3)
      while (lvl >= 3 && it[lvl] >= (lvl == 3 ? min(end3, it3n) : sz[lvl])) --lvl;
      if (lvl < 3) break;
      const uint32_t ii = it[lvl];
      __syncwarp();  // every lane has read the iterator before any lane advances it
      it[lvl] = ii + 1;
      f[lvl] = (lvl == 3 ? it3p : set[lvl])[ii];
      descend = true;
    }
    (void)lvl;
  }
  flush(A, acc, lane);
  if (lane == 0) {
    const long long t_all = clock64() - t_start;
    if (!t_ph1) t_ph1 = t_all;
    atomicAdd(&A.cnt[CNT_XT + 0], (unsigned long long)t_ph1);
    atomicMax(&A.cnt[CNT_XT + 1], (unsigned long long)t_ph1);
    atomicMax(&A.cnt[CNT_XT + 2], (unsigned long long)t_all);
    atomicMax(&A.cnt[CNT_XT + 3], (unsigned long long)t_emax);
#pragma unroll
    for (int i = 0; i < 5; ++i) atomicMax(&A.cnt[CNT_XT + 4 + i], (unsigned long long)tpm[i]);
    atomicAdd(&A.cnt[CNT_X_ENTRIES], x_entries);
    atomicAdd(&A.cnt[CNT_X_PRUNED], x_pruned);
    atomicAdd(&A.cnt[CNT_X_L3], x_l3);
    atomicAdd(&A.cnt[CNT_X_L4], x_l4);
    atomicAdd(&A.cnt[CNT_X_LAST], x_last);
    atomicAdd(&A.cnt[CNT_X_L3F], x_l3f);
  }
}

// ---- k = 4 count mode: the last level as one lean kernel ("k_last4") -------------------------
// Every level-2 frontier entry (unit, x2) of a 4-vertex query needs one count: |∩ of position 3's backward lists|
// under the entry's views, label, injectivity and symmetry range. The generic DFS kernel carries stacks, list
// arrays indexed at run time (local memory) and a chain of dependent metadata loads per entry; here
//   * the plan's position-3 rule is packed into one int4 per plan in shared memory (bit masks over positions
//     0..2: no run-time-indexed arrays, so everything stays in registers);
//   * a warp grabs up to 32 x2-grouped entries and each lane prefetches ONE entry's metadata (frontier slot,
//     unit, descriptors and delta records of its seed-side lists) in parallel, parked in a per-warp shared
//     record: the per-entry dependent global-load chain becomes one parallel round per grab;
//   * the run's x2 list is pinned once per run (shared memory, else HBM scratch for zero-copy lists);
//   * symmetry ranges trim sorted lists by a 32-way warp-parallel lower bound (2-3 ballot rounds instead of
//     log2 L dependent loads by every lane);
//   * the count is a merge path (both runs device-resident, when cheaper) or lane-parallel binary-search probes.
struct LR {
  const int32_t *m;  // main run (trimmed in place)
  uint32_t ml;
  const int32_t *x;  // delta run (device memory) or nullptr
  uint32_t xl;
  bool dev;
};

__device__ __forceinline__ uint32_t warp_lb(const int32_t *a, uint32_t n, int32_t v, int lane) {
  uint32_t lo = 0, hi = n;
  while (hi - lo > 32) {
    const uint32_t step = (hi - lo + 31) >> 5;
    const uint32_t p = lo + (uint32_t)lane * step;
    const bool pr = p < hi && a[p] < v;
    const uint32_t c = __popc(__ballot_sync(kFull, pr));
    if (c == 0) return lo;  // a[lo] >= v
    const uint32_t nlo = lo + (c - 1) * step + 1;
    hi = min(hi, lo + c * step);
    lo = nlo;
  }
  const bool pr = lo + (uint32_t)lane < hi && a[lo + lane] < v;
  return lo + __popc(__ballot_sync(kFull, pr));
}

__device__ __forceinline__ void warp_trim(LR &L, int32_t vlo, int32_t vhi, int lane) {
  if (L.ml == 0) return;
  const uint32_t b = vlo == INT_MIN ? 0u : warp_lb(L.m, L.ml, vlo + 1, lane);
  const uint32_t e = vhi == INT_MAX ? L.ml : warp_lb(L.m, L.ml, vhi, lane);
  L.m += b;
  L.ml = e > b ? e - b : 0u;
}

__device__ __forceinline__ bool lr_has(const LR &L, int32_t v) {
  return bsearch_has(L.m, L.ml, v) || (L.xl != 0 && bsearch_has(L.x, L.xl, v));
}

// pack position 3 of a k = 4 plan: x = list_mask | probe_mask << 3 | reuse << 6 | inj << 8 | lo << 11 | hi << 14 |
// kind << 17 | view(p) << (20 + 2p); y = label
__device__ int4 pack_last4(const DevPlan &P) {
  const LevelPlan &L = P.lv[3];
  unsigned lm = 0, pm = 0, im = 0, lo = 0, hi = 0, vw = 0;
  for (int b = 0; b < L.nb; ++b) {
    lm |= 1u << L.bpos[b];
    vw |= (unsigned)L.bview[b] << (2 * L.bpos[b]);
  }
  if (L.reuse >= 0)
    for (int r = 0; r < L.nrest; ++r) pm |= 1u << L.bpos[L.rest[r]];
  for (int i = 0; i < L.ninj; ++i) im |= 1u << L.inj[i];
  for (int i = 0; i < L.nlo; ++i) lo |= 1u << L.lo[i];
  for (int i = 0; i < L.nhi; ++i) hi |= 1u << L.hi[i];
  const unsigned x = lm | pm << 3 | (L.reuse >= 0 ? 1u : 0u) << 6 | im << 8 | lo << 11 | hi << 14 |
                     (unsigned)P.kind << 17 | vw << 20;
  return make_int4((int)x, L.label, 0, 0);
}

// Prefetch side: vertex v's raw descriptor with the delta run of view vw resolved -> {ptr lo, ptr hi, len, xoff}
// and the delta length in *xl.
__device__ __forceinline__ int4 lr_fetch(const MatchArgs &A, int32_t v, int vw, int *xl) {
  int4 raw = __ldg(reinterpret_cast<const int4 *>(A.vdesc + v));
  const uint32_t upd = (uint32_t)raw.w;
  *xl = 0;
  raw.w = 0;
  if (upd != 0 && vw != VIEW_S) {
    const int4 e = __ldg(reinterpret_cast<const int4 *>(A.drec + (upd - 1)));
    raw.w = vw == VIEW_NEW ? e.x : e.z;
    *xl = vw == VIEW_NEW ? e.y : e.w;
  }
  return raw;
}

// Entry side: the list from a prefetched record; algorithmic bytes accounted (hit / miss / delta).
__device__ __forceinline__ LR lr_make(const MatchArgs &A, const int4 r, int xl, Acc &acc) {
  LR l;
  l.m = reinterpret_cast<const int32_t *>((unsigned long long)(unsigned)r.x | ((unsigned long long)(unsigned)r.y << 32));
  l.ml = (uint32_t)r.z;
  l.x = xl ? A.dlist + r.w : nullptr;
  l.xl = (uint32_t)xl;
  const char *c = reinterpret_cast<const char *>(l.m);
  const bool in_ubuf = c >= A.ubuf_lo && c < A.ubuf_hi;
  l.dev = is_hit(A, l.m);
  if (in_ubuf) acc.stat(kSDelta, 4ull * l.ml);
  else if (l.dev) acc.stat(kSHit, 4ull * l.ml);
  else acc.stat(kSMiss, 4ull * l.ml);
  acc.stat(kSDelta, 4ull * l.xl);
  return l;
}

// bulk-copy a zero-copy list when the staging rule of stage_lists says so (drv: always), into the free part of
// the warp's shared slice, else its HBM staging buffer (out of line: rare, and its copy loop is register-hungry)
__device__ __noinline__ uint32_t stage_slow(LR &L, bool drv, uint32_t d, int32_t *&sm, uint32_t &sm_left,
                                            int32_t *&g, uint32_t &g_left, int lane) {  // returns the bytes copied
  const uint32_t n = L.ml;
  if (!drv) {
    const uint32_t lg = 32u - __clz(n);
    if (4ull * n > 32ull * d * (lg > 4 ? lg - 3 : 1)) return 0;
  }
  // a trimmed run starts anywhere: copy from its 16-byte granule (lists are allocated in granules)
  const uint32_t mis = (uint32_t)((reinterpret_cast<uintptr_t>(L.m) >> 2) & 3u);
  const uint32_t cn = n + mis, n4 = (cn + 3) & ~3u;
  int32_t *dst;
  if (n4 <= sm_left) {
    dst = sm;
    sm += n4;
    sm_left -= n4;
  } else if (n4 <= g_left) {
    dst = g;
    g += n4;
    g_left -= n4;
  } else {
    return 0;
  }
  warp_copy(dst, L.m - mis, cn, lane);
  __syncwarp();
  L.m = dst + mis;
  L.dev = true;
  return 4u * cn;
}

__device__ __forceinline__ void stage_one(LR &L, bool drv, uint32_t d, int32_t *&sm, uint32_t &sm_left,
                                          int32_t *&g, uint32_t &g_left, int lane, Acc &acc) {
  if (L.dev || L.ml < 32) return;
  acc.stat(kSCopied, stage_slow(L, drv, d, sm, sm_left, g, g_left, lane));
}

__device__ __noinline__ void copy_list(int32_t *dst, const int32_t *src, uint32_t n, int lane) {
  warp_copy(dst, src, n, lane);
  __syncwarp();
}

__device__ __forceinline__ uint32_t warp_sum(uint32_t c) {
#pragma unroll
  for (int o = 16; o; o >>= 1) c += __shfl_xor_sync(kFull, c, o);
  return c;
}

__device__ __forceinline__ void swap_lr(LR &a, LR &b) {
  const LR t = a;
  a = b;
  b = t;
}

// position 3's symmetry range of a packed plan for the partial match (a, b, x2); false if the plan's position 3
// does not read x2's list
__device__ __forceinline__ bool l4_range(unsigned pk, int32_t a, int32_t b, int32_t x2, int32_t *lo, int32_t *hi) {
  const bool reuse = (pk >> 6) & 1u;
  const unsigned need = reuse ? (pk >> 3) & 7u : pk & 7u;
  const unsigned lom = (pk >> 11) & 7u, him = (pk >> 14) & 7u;
  int32_t vlo = INT_MIN, vhi = INT_MAX;
  if (lom & 1u) vlo = max(vlo, a);
  if (lom & 2u) vlo = max(vlo, b);
  if (lom & 4u) vlo = max(vlo, x2);
  if (him & 1u) vhi = min(vhi, a);
  if (him & 2u) vhi = min(vhi, b);
  if (him & 4u) vhi = min(vhi, x2);
  *lo = vlo;
  *hi = vhi;
  return (need & 4u) != 0;
}

#ifndef GCSM_PIN_RANGE
#define GCSM_PIN_RANGE 0  // 1: pin only the run's symmetry-range slice of x2's list (search costs > bytes saved)
#endif
#ifndef GCSM_ZC_TRIM
#define GCSM_ZC_TRIM 0
#endif
#ifndef GCSM_L4_MINBLOCKS
#define GCSM_L4_MINBLOCKS 3
#endif
#ifndef GCSM_LAST4
#define GCSM_LAST4 1
#endif
constexpr int kL4Meta = 32 * 4;  // int4 per warp: 32 entries x 4
constexpr int kL4SmemBytes = kSmemBytes + kWarps * kL4Meta * 16 + GCSM_MAXPLANS * 16;

__global__ void __launch_bounds__(kBlock, GCSM_L4_MINBLOCKS) k_last4(const __grid_constant__ MatchArgs A) {
  const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  extern __shared__ int4 smem_raw[];
  int32_t *sm = reinterpret_cast<int32_t *>(smem_raw) + wib * kSmemInts;
  int4 *meta = smem_raw + kSmemBytes / 16 + wib * kL4Meta;
  int4 *lp = smem_raw + kSmemBytes / 16 + kWarps * kL4Meta;
  for (int i = threadIdx.x; i < A.n_plans; i += blockDim.x) lp[i] = pack_last4(A.plans[i]);
  __syncthreads();
  int32_t *gstage = A.scratch + gw * A.scratch_stride + A.scratch_stride - 2 * (int64_t)A.dcap;
  int32_t *pstage = gstage - (int64_t)A.dcap;
  const int64_t n_f2 = (int64_t)*(volatile unsigned long long *)&A.cnt[CNT_F2];
  const int32_t *f2c = reinterpret_cast<const int32_t *>(A.f2);
  const int32_t *f2u = f2c + A.f2_cap;
  const int64_t warps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  // work grab: up to GCSM_L4_GRAB entries (rounds of 32), fewer when the frontier would leave warps idle. A run of
  // entries sharing x2 is cut only at grab boundaries, where its zero-copy list is fetched again.
  const int64_t chunk = max((int64_t)1, min((int64_t)GCSM_L4_GRAB, n_f2 / (8 * warps)));
  __shared__ unsigned long long s_stats[kWarps][kSN];
  Acc acc;
  acc.init(s_stats[wib], lane);
  unsigned long long d_runs = 0, d_pinb = 0, d_pins = 0, d_split = 0;
  for (;;) {
    unsigned long long g0 = 0;
    if (lane == 0) g0 = atomicAdd(&A.cnt[CNT_CURSOR1], (unsigned long long)chunk);
    g0 = __shfl_sync(kFull, g0, 0);
    if ((int64_t)g0 >= n_f2) break;
    const int64_t gend = min((int64_t)g0 + chunk, n_f2);
    int32_t pin_v = -1;  // x2 of the current run and its list slice (pinned copy, or in place): kept across rounds
    const int32_t *pin_p = nullptr;
    uint32_t pin_len = 0;
    int4 xraw = make_int4(0, 0, 0, 0);
    int4 xrec = make_int4(0, 0, 0, 0);  // x2's delta record (if updated)
    uint32_t pin_sm = 0;
    bool pin_dev = false, pin_hit = false, pin_peer = false;
    for (int64_t c0 = (int64_t)g0; c0 < gend; c0 += 32) {
    const int n = (int)min((int64_t)32, gend - c0);
    // ---- one lane per entry: prefetch the entry's metadata in parallel
    __syncwarp();
    if (lane < n) {
      const int64_t j = (int64_t)c0 + lane;
      const int64_t e = A.group ? A.group[j] : j;
      const int32_t x2 = f2c[e], ui = f2u[e];
      const int4 u = __ldg(reinterpret_cast<const int4 *>(A.units + ui));  // a, b, plan
      const unsigned pk = (unsigned)lp[u.z].x;
      const unsigned need = (pk >> 6) & 1u ? (pk >> 3) & 7u : pk & 7u;
      int4 r1 = make_int4(0, 0, 0, 0), r2 = make_int4(0, 0, 0, 0);
      int2 seg = make_int2(0, 0);
      int xl0 = 0, xl1 = 0;
      if (need & 1u) {
        r1 = lr_fetch(A, u.x, (pk >> 20) & 3u, &xl0);
        mark_touched(A, u.x);
      }
      if (need & 2u) {
        r2 = lr_fetch(A, u.y, (pk >> 22) & 3u, &xl1);
        mark_touched(A, u.y);
      }
      if ((pk >> 6) & 1u) seg = A.useg[ui];
      meta[4 * lane + 0] = make_int4(x2, u.z, u.x, u.y);
      meta[4 * lane + 1] = r1;
      meta[4 * lane + 2] = r2;
      meta[4 * lane + 3] = make_int4(seg.x, seg.y, xl0, xl1);
    }
    __syncwarp();
    for (int i = 0; i < n; ++i) {
      const int4 m0 = meta[4 * i];
      const int32_t x2 = m0.x, a = m0.z, b = m0.w;
      if (x2 != pin_v) {  // new run: entries i..i+run-1 share x2 (it may continue into the grab's next rounds)
        const int64_t jn = c0 + i + 1 + lane;
        const bool same = jn < gend && f2c[A.group ? A.group[jn] : jn] == x2;
        const unsigned rm = __ballot_sync(kFull, same);
        const int run = 1 + (rm == kFull ? 32 : __ffs(~rm) - 1);
        // union of the symmetry ranges of the run's entries that read x2's list: only that slice is fetched
        // (entries of later rounds are not prefetched yet: then the whole list)
        int32_t rlo = INT_MAX, rhi = INT_MIN;
        if (i + run > n) {
          rlo = INT_MIN;
          rhi = INT_MAX;
        } else if (lane < run) {
          const int4 mr = meta[4 * (i + lane)];
          int32_t lo, hi;
          if (l4_range((unsigned)lp[mr.y].x, mr.z, mr.w, x2, &lo, &hi)) {
            rlo = lo;
            rhi = hi;
          }
        }
        rlo = __reduce_min_sync(kFull, rlo);
        rhi = __reduce_max_sync(kFull, rhi);
        pin_v = x2;
        if (lane == 0 && rlo <= rhi) mark_touched(A, x2);
        xraw = __ldg(reinterpret_cast<const int4 *>(A.vdesc + x2));
        xrec = xraw.w ? __ldg(reinterpret_cast<const int4 *>(A.drec + ((uint32_t)xraw.w - 1))) : make_int4(0, 0, 0, 0);
        const int32_t *mp = reinterpret_cast<const int32_t *>((unsigned long long)(unsigned)xraw.x |
                                                                ((unsigned long long)(unsigned)xraw.y << 32));
        const uint32_t ml = (uint32_t)xraw.z;
        pin_hit = is_hit(A, mp);
        pin_peer = false;
        if (!pin_hit && A.npeer && xraw.w == 0 && ml > 0) {  // a linked peer's HBM cache holds x2's list
          const int32_t *q = peer_lookup(A, x2, ml);
          if (q) {
            mp = q;
            pin_hit = true;
            pin_peer = true;
          }
        }
        uint32_t lb = 0, le = ml;
        if (rlo > rhi) {
          le = 0;  // no entry of the run reads x2's list
        } else if (!pin_hit && A.sidx && ml >= 64 && (rlo != INT_MIN || rhi != INT_MAX) &&
                   __ldg(A.soff + x2) != 0xffffffffu) {
          // zero-copy list with a sampled index in HBM (every 32nd element): the run's symmetry-range slice is
          // located without touching host memory and only that slice crosses PCIe (32-element granularity;
          // every read below is range-checked or range-trimmed)
          const int32_t *smp = A.sidx + __ldg(A.soff + x2);
          const uint32_t ns = (ml + 31) >> 5;
          if (rlo != INT_MIN) {
            const uint32_t j = warp_lb(smp, ns, rlo + 1, lane);  // samples <= rlo
            lb = j ? 32u * (j - 1) : 0u;
          }
          if (rhi != INT_MAX) {
            const uint32_t j = warp_lb(smp, ns, rhi, lane);  // samples < rhi: list[32 j] >= rhi when j < ns
            le = max(lb, min(ml, 32u * j));
          }
        } else if (GCSM_PIN_RANGE && ml >= 32) {
          if (rlo != INT_MIN) lb = warp_lb(mp, ml, rlo + 1, lane);
          if (rhi != INT_MAX) le = max(lb, warp_lb(mp, ml, rhi, lane));
        }
        pin_p = mp + lb;
        pin_len = le - lb;
        pin_dev = pin_hit;
        pin_sm = 0;
        ++d_runs;
        // copy from the 16-byte granule holding the slice's first element (lists are granule-aligned)
        const uint32_t mis = lb & 3u, cn = pin_len + mis, cn4 = (cn + 3) & ~3u;
        if (run >= 2 && pin_len >= 32 && !pin_hit) {
          ++d_pins;
          d_pinb += 4ull * cn;
          // GCSM_TRACE: a run continuing the previous grab's run (same x2 across the grab boundary) fetches again
          if (i == 0 && c0 == (int64_t)g0 && c0 > 0 && f2c[A.group ? A.group[c0 - 1] : c0 - 1] == x2) d_split += 4ull * cn;
        }
        if (run >= 2 && pin_len >= 32 && cn4 <= GCSM_PIN_SMEM_MAX) {
          copy_list(sm, mp + (lb - mis), cn, lane);
          if (!pin_hit) acc.stat(kSCopied, 4ull * cn);
          pin_p = sm + mis;
          pin_dev = true;
          pin_sm = cn4;
        } else if (run >= 2 && pin_len >= 32 && !pin_hit) {
          copy_list(pstage, mp + (lb - mis), cn, lane);
          acc.stat(kSCopied, 4ull * cn);
          pin_p = pstage + mis;
          pin_dev = true;
        }
      }
      const unsigned pk = (unsigned)lp[m0.y].x;
      const int label = lp[m0.y].y;
      const bool reuse = (pk >> 6) & 1u;
      const unsigned need = reuse ? (pk >> 3) & 7u : pk & 7u;
      const unsigned im = (pk >> 8) & 7u, lom = (pk >> 11) & 7u, him = (pk >> 14) & 7u;
      const int kind = (pk >> 17) & 1u;
      int32_t vlo = INT_MIN, vhi = INT_MAX;
      if (lom & 1u) vlo = max(vlo, a);
      if (lom & 2u) vlo = max(vlo, b);
      if (lom & 4u) vlo = max(vlo, x2);
      if (him & 1u) vhi = min(vhi, a);
      if (him & 2u) vhi = min(vhi, b);
      if (him & 4u) vhi = min(vhi, x2);
      const int32_t ex0 = (im & 1u) ? a : -1, ex1 = (im & 2u) ? b : -1, ex2 = (im & 4u) ? x2 : -1;
      // the lists: slot 0 = driver, slots 1.. = probes (positions in ascending order; selects, no indexed arrays)
      const int4 m3 = meta[4 * i + 3];
      LR La, Lb, Lc;
      La.xl = Lb.xl = Lc.xl = 0;
      La.x = Lb.x = Lc.x = nullptr;
      La.ml = Lb.ml = Lc.ml = 0;
      La.m = Lb.m = Lc.m = nullptr;
      La.dev = Lb.dev = Lc.dev = true;
      if (need & 1u) La = lr_make(A, meta[4 * i + 1], m3.z, acc);
      if (need & 2u) Lb = lr_make(A, meta[4 * i + 2], m3.w, acc);
      if (need & 4u) {
        const int vw = (pk >> 24) & 3u;
        Lc.m = pin_p;
        Lc.ml = pin_len;  // the run's range slice (every read below is range-checked or range-trimmed)
        Lc.dev = pin_dev;
        if (xraw.w != 0 && vw != VIEW_S) {
          Lc.x = A.dlist + (vw == VIEW_NEW ? xrec.x : xrec.z);
          Lc.xl = (uint32_t)(vw == VIEW_NEW ? xrec.y : xrec.w);
        }
        if (pin_hit && !pin_peer) acc.stat(kSHit, 4ull * (uint32_t)xraw.z);  // algorithmic: the whole list
        else acc.stat(kSMiss, 4ull * (uint32_t)xraw.z);
        if (pin_peer) acc.stat(kSPeer, 4ull * (uint32_t)xraw.z);
        acc.stat(kSDelta, 4ull * Lc.xl);
      }
      const LR first = (need & 1u) ? La : ((need & 2u) ? Lb : Lc);
      const LR second = (need & 1u) ? ((need & 2u) ? Lb : Lc) : Lc;
      const int nl = __popc(need) + (reuse ? 1 : 0);
      LR L0, L1, L2;
      if (reuse) {  // the unit's level-2 candidate set (code motion); not globally sorted (main then delta run)
        L0.m = f2c + m3.x;
        L0.ml = (uint32_t)m3.y;
        L0.x = nullptr;
        L0.xl = 0;
        L0.dev = true;
        L1 = first;
        L2 = second;
      } else {
        L0 = first;
        L1 = second;
        L2 = Lc;
      }
#if GCSM_ZC_TRIM
      // zero-copy lists: only their range slice is read and staged (costs PCIe round trips: measured slower)
      if (!L0.dev && L0.ml >= 32) warp_trim(L0, vlo, vhi, lane);
      if (nl >= 2 && !L1.dev && L1.ml >= 32) warp_trim(L1, vlo, vhi, lane);
      if (nl >= 3 && !L2.dev && L2.ml >= 32) warp_trim(L2, vlo, vhi, lane);
#endif
      if (!reuse) {  // the smallest list drives
        if (nl >= 2 && L1.ml + L1.xl < L0.ml + L0.xl) swap_lr(L0, L1);
        if (nl >= 3 && L2.ml + L2.xl < L0.ml + L0.xl) swap_lr(L0, L2);
      }
      const uint32_t d = L0.ml + L0.xl;
      int32_t *smf = sm + pin_sm, *gf = gstage;
      uint32_t sml = kSmemInts - pin_sm, gl = 2u * (uint32_t)A.dcap;
      stage_one(L0, true, d, smf, sml, gf, gl, lane, acc);
      if (nl >= 2) stage_one(L1, false, d, smf, sml, gf, gl, lane, acc);
      if (nl >= 3) stage_one(L2, false, d, smf, sml, gf, gl, lane, acc);
      uint32_t c = 0;
      bool done = false;
      if (!reuse && nl == 2 && L0.dev && L1.dev && L0.ml >= 8 && L1.ml >= 8) {
        // merge path on the range-trimmed main runs when cheaper than d/32 rounds of binary search
        warp_trim(L0, vlo, vhi, lane);
        warp_trim(L1, vlo, vhi, lane);
        const uint32_t dd = L0.ml + L0.xl, big = L1.ml + L1.xl;
        const uint32_t bs_cost = ((dd + 31) >> 5) * (7 * ilog2(big) + 12);
        const uint32_t mg_cost = 10 * ilog2(min(L0.ml, L1.ml) | 1u) + 7 * ((L0.ml + L1.ml + 31) >> 5) + 30;
        if (mg_cost < bs_cost && L0.ml > 0 && L1.ml > 0) {
          c = merge_count(L0.m, L0.ml, L1.m, L1.ml, label, A.lab, lane);
          if (L0.xl) c += probe_count(L0.x, L0.xl, L1.m, L1.ml, label, A.lab, lane, vlo, vhi);
          if (L1.xl) c += probe_count(L1.x, L1.xl, L0.m, L0.ml, label, A.lab, lane, vlo, vhi);
          if (L0.xl && L1.xl) c += probe_count(L0.x, L0.xl, L1.x, L1.xl, label, A.lab, lane, vlo, vhi);
          const int32_t exs[3] = {ex0, ex1, ex2};
#pragma unroll
          for (int q = 0; q < 3; ++q) {
            const int32_t v = exs[q];
            if (v >= 0 && v > vlo && v < vhi && (label < 0 || A.lab[v] == (uint16_t)label) && lr_has(L0, v) &&
                lr_has(L1, v))
              --c;
          }
          done = true;
        }
      } else if (L0.dev && !reuse) {
        warp_trim(L0, vlo, vhi, lane);
      }
      if (!done) {
        if (nl == 1 && label < 0 && !reuse) {  // single list: its in-range size minus the excluded vertices it holds
          uint32_t cx = 0;
          for (uint32_t q = lane; q < L0.xl; q += 32) {
            const int32_t v = L0.x[q];
            cx += v > vlo && v < vhi;
          }
          c = (L0.dev ? L0.ml : 0u) + warp_sum(cx);
          if (!L0.dev) {  // untrimmed zero-copy run: count in range
            uint32_t cm = 0;
            for (uint32_t q = lane; q < L0.ml; q += 32) {
              const int32_t v = L0.m[q];
              cm += v > vlo && v < vhi;
            }
            c += warp_sum(cm);
          }
          const int32_t exs[3] = {ex0, ex1, ex2};
#pragma unroll
          for (int q = 0; q < 3; ++q) {
            const int32_t v = exs[q];
            if (v >= 0 && v > vlo && v < vhi && lr_has(L0, v)) --c;
          }
        } else {  // lane-parallel probes of the driver's elements
          uint32_t cnt = 0;
          const uint32_t total = L0.ml + L0.xl;
          for (uint32_t q = lane; q < total; q += 32) {
            const int32_t v = q < L0.ml ? L0.m[q] : L0.x[q - L0.ml];
            bool ok = v > vlo && v < vhi && v != ex0 && v != ex1 && v != ex2;
            if (ok && nl >= 2) ok = lr_has(L1, v);
            if (ok && nl >= 3) ok = lr_has(L2, v);
            if (ok && label >= 0) ok = A.lab[v] == (uint16_t)label;
            cnt += ok;
          }
          c = warp_sum(cnt);
        }
      }
      if (kind) acc.rem += c;
      else acc.add += c;
    }
    }
  }
  flush(A, acc, lane);
  if (lane == 0) {
    atomicAdd(&A.cnt[CNT_DBG_RUNS], d_runs);
    atomicAdd(&A.cnt[CNT_DBG_PINBYTES], d_pinb);
    atomicAdd(&A.cnt[CNT_DBG_PINS], d_pins);
    atomicAdd(&A.cnt[CNT_DBG_SPLIT], d_split);
  }
}

// ---- counting sort of the level-2 frontier by its candidate vertex x2 (entries sharing x2 are
// processed back to back by one warp, which stages x2's zero-copy list once per run).
__global__ void k_group_hist(const int32_t *f2c, const unsigned long long *cnt, uint32_t *hist) {
  const int64_t n = (int64_t)cnt[CNT_F2];
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < n; e += (int64_t)gridDim.x * blockDim.x)
    atomicAdd(&hist[f2c[e]], 1u);
}

constexpr int kScanItems = 8;  // per thread, 256 threads: 2048 per block

// in-place exclusive scan of a[0..n) per 2048-block; block totals to bsum
__global__ void k_scan_local(uint32_t *a, int64_t n, uint32_t *bsum) {
  __shared__ uint32_t ws[8];
  const int64_t base = (int64_t)blockIdx.x * 2048 + threadIdx.x * kScanItems;
  uint32_t v[kScanItems], run = 0;
  for (int i = 0; i < kScanItems; ++i) {
    v[i] = base + i < n ? a[base + i] : 0u;
    const uint32_t t = v[i];
    v[i] = run;
    run += t;
  }
  // exclusive scan of the per-thread totals across the block
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  uint32_t x = run;
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t y = __shfl_up_sync(kFull, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) ws[w] = x;
  __syncthreads();
  if (w == 0) {
    uint32_t t = lane < 8 ? ws[lane] : 0u;
    for (int o = 1; o < 8; o <<= 1) {
      const uint32_t y = __shfl_up_sync(kFull, t, o);
      if (lane >= o) t += y;
    }
    if (lane < 8) ws[lane] = t;
  }
  __syncthreads();
  const uint32_t excl = x - run + (w ? ws[w - 1] : 0u);
  for (int i = 0; i < kScanItems; ++i)
    if (base + i < n) a[base + i] = v[i] + excl;
  if (threadIdx.x == 255) bsum[blockIdx.x] = excl + run;
}

// single block: exclusive scan of the block totals (loops for any count)
__global__ void k_scan_bsum(uint32_t *bsum, int64_t nb) {
  __shared__ uint32_t carry;
  if (threadIdx.x == 0) carry = 0;
  __syncthreads();
  for (int64_t s0 = 0; s0 < nb; s0 += 1024) {
    const int64_t i = s0 + threadIdx.x;
    const uint32_t v = i < nb ? bsum[i] : 0u;
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    uint32_t x = v;
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(kFull, x, o);
      if (lane >= o) x += y;
    }
    __shared__ uint32_t ws[32];
    if (lane == 31) ws[w] = x;
    __syncthreads();
    if (w == 0) {
      uint32_t t = ws[lane];
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(kFull, t, o);
        if (lane >= o) t += y;
      }
      ws[lane] = t;
    }
    __syncthreads();
    const uint32_t incl = x + (w ? ws[w - 1] : 0u);
    if (i < nb) bsum[i] = carry + incl - v;
    __syncthreads();
    if (threadIdx.x == 1023) carry += incl;
    __syncthreads();
  }
}

__global__ void k_scan_add(uint32_t *a, int64_t n, const uint32_t *bsum) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    a[i] += bsum[i / 2048];
}

__global__ void k_group_scatter(const int32_t *f2c, const unsigned long long *cnt, uint32_t *cursor,
                                int32_t *group) {
  const int64_t n = (int64_t)cnt[CNT_F2];
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < n; e += (int64_t)gridDim.x * blockDim.x)
    group[atomicAdd(&cursor[f2c[e]], 1u)] = (int32_t)e;
}

// Warp per cache list: copy n16 16-byte granules to dst + tri[3i+1] from src + tri[3i] (src == nullptr: tri[3i] is
// an absolute address — a mapped pinned host list pulled over PCIe; else an offset into the previous cache buffer).
__global__ void k_gather(char *dst, const char *src, const uint64_t *tri, int64_t n) {
  const int lane = threadIdx.x & 31;
  const int64_t w = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t i = w; i < n; i += nw) {
    const int4 *s4 = reinterpret_cast<const int4 *>(src ? src + tri[3 * i] : reinterpret_cast<const char *>(tri[3 * i]));
    int4 *d4 = reinterpret_cast<int4 *>(dst + tri[3 * i + 1]);
    const uint64_t n16 = tri[3 * i + 2];
    for (uint64_t base = 0; base < n16; base += 128) {  // 4 x 16 B per lane in flight
      int4 v[4];
#pragma unroll
      for (int u = 0; u < 4; ++u)
        if (base + lane + 32 * u < n16) v[u] = s4[base + lane + 32 * u];
#pragma unroll
      for (int u = 0; u < 4; ++u)
        if (base + lane + 32 * u < n16) d4[base + lane + 32 * u] = v[u];
    }
  }
}

__global__ void k_patch(VDesc *vdesc, const int64_t *idx, const VDesc *val, int64_t n) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    vdesc[idx[i]] = val[i];
}

}  // namespace

cudaError_t upload_plans(DevPlan *dst, const DevPlan *plans, int n, cudaStream_t s) {
  return cudaMemcpyAsync(dst, plans, sizeof(DevPlan) * (size_t)n, cudaMemcpyHostToDevice, s);
}

int match_grid(int device, int *warps_total) {
  int sms = 0, occ = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device);
  cudaFuncSetAttribute(k_extend<false, 0>, cudaFuncAttributeMaxDynamicSharedMemorySize, kExtSmemBytes);
  cudaFuncSetAttribute(k_extend<false, 4>, cudaFuncAttributeMaxDynamicSharedMemorySize, kExtSmemBytes);
  cudaFuncSetAttribute(k_extend<true, 0>, cudaFuncAttributeMaxDynamicSharedMemorySize, kExtSmemBytes);
  cudaFuncSetAttribute(k_level2<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, kSmemBytes);
  cudaFuncSetAttribute(k_level2<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, kSmemBytes);
  cudaFuncSetAttribute(k_last4, cudaFuncAttributeMaxDynamicSharedMemorySize, kL4SmemBytes);
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_extend<false, 0>, kBlock, kExtSmemBytes);
  int occ2 = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ2, k_level2<false>, kBlock, kSmemBytes);
  if (occ2 < occ) occ = occ2;
  if (occ < 1) occ = 1;
  const int grid = sms * occ;
  if (warps_total) *warps_total = grid * kWarps;
  return grid;
}

cudaError_t launch_level2(const MatchArgs &a0, int grid, cudaStream_t s) {
  MatchArgs a = a0;
  a.acc_base = CNT_ACC_L2;
  a.stage_state = nullptr;  // level 2 reads the seeds' lists (the batch's uploaded U lists on the GPU path)
  if (a.listing) k_level2<true><<<grid, kBlock, kSmemBytes, s>>>(a);
  else k_level2<false><<<grid, kBlock, kSmemBytes, s>>>(a);
  return cudaGetLastError();
}

__global__ void k_reset_sharing(unsigned long long *cnt) {
  cnt[CNT_ARENA] = 0;
  cnt[CNT_TAIL] = 0;
  cnt[CNT_HEAD] = 0;
  cnt[CNT_PRODUCERS] = 0;
}

cudaError_t launch_extend(const MatchArgs &a0, int grid, cudaStream_t s) {
  MatchArgs a = a0;
  a.acc_base = CNT_ACC_EXT;
  if (a.tasks) k_reset_sharing<<<1, 1, 0, s>>>(a.cnt);
  if (a.listing) k_extend<true, 0><<<grid, kBlock, kExtSmemBytes, s>>>(a);
  else if (a.k == 4 && GCSM_LAST4) k_last4<<<grid, kBlock, kL4SmemBytes, s>>>(a);
  else if (a.k == 4) k_extend<false, 4><<<grid, kBlock, kExtSmemBytes, s>>>(a);
  else k_extend<false, 0><<<grid, kBlock, kExtSmemBytes, s>>>(a);
  return cudaGetLastError();
}

cudaError_t launch_group_frontier(const MatchArgs &a, int32_t n_vertices, uint32_t *hist, uint32_t *bsum,
                                  int32_t *group, cudaStream_t s) {
  const int32_t *f2c = reinterpret_cast<const int32_t *>(a.f2);
  cudaError_t e = cudaMemsetAsync(hist, 0, sizeof(uint32_t) * (size_t)n_vertices, s);
  if (e != cudaSuccess) return e;
  k_group_hist<<<148 * 8, 256, 0, s>>>(f2c, a.cnt, hist);
  const int64_t nb = ((int64_t)n_vertices + 2047) / 2048;
  k_scan_local<<<(unsigned)nb, 256, 0, s>>>(hist, n_vertices, bsum);
  k_scan_bsum<<<1, 1024, 0, s>>>(bsum, nb);
  k_scan_add<<<148 * 8, 256, 0, s>>>(hist, n_vertices, bsum);
  k_group_scatter<<<148 * 8, 256, 0, s>>>(f2c, a.cnt, hist, group);
  return cudaGetLastError();
}

cudaError_t launch_gather_lists(char *dst, const char *src, const uint64_t *tri, int64_t n, cudaStream_t s) {
  if (n <= 0) return cudaSuccess;
  const int grid = (int)std::min<int64_t>((n + 7) / 8, 148 * 16);
  k_gather<<<grid, 256, 0, s>>>(dst, src, tri, n);
  return cudaGetLastError();
}

__global__ void k_sidx_update(int32_t *sidx, uint32_t *soff, const int4 *rec, int64_t n, const int32_t *staged) {
  const int lane = threadIdx.x & 31;
  for (int64_t i = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; i < n;
       i += ((int64_t)gridDim.x * blockDim.x) >> 5) {
    const int4 r = rec[i];  // vertex, offset (or -1), count, staging position
    if (r.y >= 0)
      for (int j = lane; j < r.z; j += 32) sidx[(uint32_t)r.y + j] = staged[(uint32_t)r.w + j];
    if (lane == 0) soff[r.x] = r.y >= 0 ? (uint32_t)r.y : 0xffffffffu;
  }
}

cudaError_t launch_sidx_update(int32_t *sidx, uint32_t *soff, const int4 *rec, int64_t n, const int32_t *staged,
                               cudaStream_t s) {
  if (n <= 0) return cudaSuccess;
  const int grid = (int)std::min<int64_t>((n + 7) / 8, 148 * 8);
  k_sidx_update<<<grid, 256, 0, s>>>(sidx, soff, rec, n, staged);
  return cudaGetLastError();
}

__global__ void k_bcomp(const uint32_t *touched, int32_t n, const VDesc *vdesc, const char *cache_lo,
                        const char *cache_hi, const char *ubuf_lo, const char *ubuf_hi, unsigned long long *out) {
  unsigned long long b[3] = {0, 0, 0};
  const int64_t W = ((int64_t)n + 31) >> 5;
  for (int64_t w = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; w < W; w += (int64_t)gridDim.x * blockDim.x) {
    uint32_t bits = touched[w];
    while (bits) {
      const int i = __ffs(bits) - 1;
      bits &= bits - 1;
      const VDesc d = vdesc[w * 32 + i];
      const char *p = reinterpret_cast<const char *>(d.ptr);
      const int where = (p >= cache_lo && p < cache_hi) ? 0 : ((p >= ubuf_lo && p < ubuf_hi) ? 2 : 1);
      b[where] += 4ull * d.len;
    }
  }
  for (int j = 0; j < 3; ++j) {
    unsigned long long x = b[j];
    for (int o = 16; o; o >>= 1) x += __shfl_xor_sync(kFull, x, o);
    if ((threadIdx.x & 31) == 0 && x) atomicAdd(out + j, x);
  }
}

cudaError_t launch_bcomp(const uint32_t *touched, int32_t n, const VDesc *vdesc, const char *cache_lo,
                         const char *cache_hi, const char *ubuf_lo, const char *ubuf_hi, unsigned long long *out,
                         cudaStream_t s) {
  k_bcomp<<<148 * 4, 256, 0, s>>>(touched, n, vdesc, cache_lo, cache_hi, ubuf_lo, ubuf_hi, out);
  return cudaGetLastError();
}

cudaError_t launch_patch_vdesc(VDesc *vdesc, const int64_t *idx, const VDesc *val, int64_t n, cudaStream_t s) {
  if (n <= 0) return cudaSuccess;
  int grid = (int)std::min<int64_t>((n + 255) / 256, 148 * 8);
  k_patch<<<grid, 256, 0, s>>>(vdesc, idx, val, n);
  return cudaGetLastError();
}

}  // namespace gcsm
