// estimator_gpu.cuh — launch interface of the GPU estimator and cache packer (steps ② and ③ on sm_100a).
//
// The paper runs the random walks on the CPU (§IV) and packs the cache on the host; here both
// run on the context's stream between the batch's uploads and its matching kernels, so the host never waits for
// the GPU inside a submit. The results are identical to the host estimator and to the oracle's `estimate` /
// `select_cache`: the same counter-based keys (R22), the same binomial algorithms (BINV / BTRD, R20) evaluated
// with the same IEEE operation sequence (explicit round-to-nearest intrinsics, no FMA contraction; the only
// transcendental, log in BTRD's rejection tests, is CUDA's ≤ 1-ulp log — see DESIGN.md), integer per-level sums,
// and the same ranking rule (R23: estimate desc, id asc, longest prefix under the budget).
#pragma once
#include <cuda_runtime.h>

#include "internal.h"
#include "stage.cuh"

namespace gcsm {

// One level-1 node of the walks: a unit with its multiplicity B_1 ~ Bin(M, 1/N1) (drawn on the host: N1 draws)
// and its key (R22 chain over seed, batch, term, kind, a, b).
struct alignas(16) EstUnit {
  int32_t a, b, plan, pad;
  unsigned long long B, key;
};

// Level-2 node of the walks (k >= 5): positions 0..2 matched, multiplicity B, key.
struct alignas(16) EstNode2 {
  int32_t f0, f1, f2, plan;
  unsigned long long B, key;
};

constexpr int kEstItem = 1024;  // level-1 driver elements per work item (a hub's children spread over warps)

struct EstQuery {
  const DevPlan *plans;     // unrestricted plans (the walks sample the paper's full trees, R27)
  const EstUnit *units;     // B > 0 only, heaviest first
  int64_t n_units;
  const int2 *items;        // (unit, first driver index): max(1, ceil(driver / kEstItem)) per unit
  int64_t n_items;
  int64_t f2_cap;           // level-2 node capacity (k >= 5): sum of the units' driver lengths
  unsigned long long *levcnt;  // dense: n x levels (zero outside the touched set)
  int32_t k;
  uint64_t N1, M;
  double powD[8];           // std::pow(D, l - 1) for l = 1..k-2 (host libm: the exact integer powers)
};

// Device-side selection state (one per context).
struct SelState {
  unsigned long long n_touched;       // vertices with a record this batch (all queries)
  unsigned long long prev_touched;    // last batch's, cleared at the start of this one
  unsigned long long prev_sel;        // vertices cached by the last batch (their descriptors point into the cache)
  unsigned long long above, prefix, mask;  // ranking cut: bytes strictly above it, score bits / mask of its bucket
  unsigned long long sel_bytes;       // cache bytes used this batch
  int32_t found;                      // 1: the budget cuts the ranking; 0: every ranked vertex fits
  int32_t err;                        // non-zero: internal error (r0 table too short)
};

struct CacheStep {
  int32_t n;                // vertex universe
  int32_t nq;
  EstQuery q[GCSM_MAX_QUERIES];
  int policy;               // 1 = estimator, 2 = degree (GCSM_CACHE_*); 0 = no cache this batch
  bool reset_first;         // descriptors of the last selection must be reset before anything reads them
  uint64_t budget;          // bytes (multiple of 16)
  // graph views
  VDesc *vdesc;             // effective descriptors (cache slot or host list)
  const unsigned long long *hptr;  // host list address of every vertex's main list
  const DRec *drec;
  const int32_t *dlist;
  const uint16_t *lab;
  // binomial tables
  double pD;                // 1 / D
  const double *r0tab;      // (1 - pD)^n for n < r0n (host std::pow)
  int64_t r0n;
  const double *sfc_dev;    // BTRD's Stirling correction for k < 10 (host lgamma), 10 doubles in device memory
  // scratch (capacity n unless noted)
  uint32_t *touched;        // ceil(n/32) words
  uint32_t *wcnt;           // ceil(n/32) + 1
  uint32_t *woff;           // ceil(n/32) + 1
  int32_t *tids;            // touched ids, ascending
  unsigned long long *bits; // score bits
  unsigned long long *bytes;
  unsigned long long *scan; // tie / offset scans
  unsigned long long *off;
  uint8_t *flag;
  int32_t *prev_sel;        // last selection (ids ascending)
  unsigned long long *hist; // 6 x 4096
  SelState *st;
  unsigned long long *cursor;  // 3 per query: item cursor, level-2 node cursor, level-2 node count
  EstNode2 *f2;             // level-2 nodes (shared by the queries, one after the other)
  void *cub_tmp;
  size_t cub_tmp_bytes;
  // cache buffers
  char *cache;              // this batch's buffer (written)
  // stats
  unsigned long long *cnt_cached;  // 3 counters: vertices, bytes, internal error
  // fetch-once staging of the walks' zero-copy lists (stage.state == nullptr: off); lists already in device memory
  // at walk time (the last batch's cache, the batch's U lists) are read in place
  cudaEvent_t *ev_walk = nullptr;  // 2 per query: around its walk kernels (timing, may be null)
  unsigned long long *alg_cnt[GCSM_MAX_QUERIES] = {};  // per query: algorithmic list bytes of its walks
  StageRef stage{};
  int32_t walk_stage = 1;  // skip-sampled drivers: 0 always staged, 1 when >= 1 selection is expected, 2 never
  int32_t walk_lane = 1;   // level k-3 nodes in BINV's domain one per lane (walk_leaf_parent)
  uint32_t stage_min = 1;
  unsigned long long *stage_cnt = nullptr;  // fill bytes, lists, hit bytes
  const char *dev_lo[2] = {nullptr, nullptr}, *dev_hi[2] = {nullptr, nullptr};
  const int32_t *sidx = nullptr;  // sampled index of the host lists (every 32nd element) and per-vertex offsets
  const uint32_t *soff = nullptr;
};

size_t cache_step_tmp_bytes(int32_t n);
cudaError_t launch_cache_step(const CacheStep &c, cudaStream_t s, uint64_t *launches);
// descriptors and host addresses of the batch's changed vertices (prev_U ∪ U)
cudaError_t launch_patch_vdesc_host(VDesc *vdesc, unsigned long long *hptr, const int64_t *idx, const VDesc *val,
                                    int64_t n, cudaStream_t s);
// the last batch's estimator output for one query: the rows of `levcnt` (levels wide) of the first n touched ids,
// into lev_out (8 per row, zero-padded); the caller drops the all-zero rows (vertices only other queries read)
cudaError_t launch_estimates_gather(const int32_t *tids, int64_t n, const unsigned long long *levcnt, int levels,
                                    unsigned long long *lev_out, cudaStream_t s);

}  // namespace gcsm
