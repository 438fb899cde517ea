// kernels.cuh — launch interface of the sm_100a matching kernels (kernels.cu).
#pragma once
#include <cuda_runtime.h>

#include "internal.h"

namespace gcsm {

// Device counters (uint64) written by the kernels.
enum Counter {
  CNT_ADDED = 0,    // embeddings found by + units
  CNT_REMOVED = 1,  // embeddings found by - units
  CNT_F2 = 4,       // level-2 frontier entries written
  CNT_OVERFLOW = 5, // frontier overflow guard (must stay 0)
  CNT_TUP_ADD = 6,  // tuples found (list mode)
  CNT_TUP_REM = 7,
  CNT_CURSOR0 = 8,  // work cursors (reset per launch)
  CNT_CURSOR1 = 9,
  CNT_DBG_SPLIT = 2,     // k_last4: bytes pinned again for runs split across work grabs (GCSM_TRACE)
  CNT_COPIED = 3,   // bytes bulk-copied from host memory by the kernels' staging (real zero-copy reads)
  // per kernel, 3 consecutive slots: list bytes (algorithmic: 4 B x list length per use) served from
  // the HBM cache, zero-copy from pinned host memory, and from the device delta segments (ins/del of U)
  CNT_ACC_L2 = 10,
  CNT_ACC_EXT = 13,
  CNT_ARENA = 16,   // ints used in the level-3 task arena
  CNT_TAIL = 17,    // level-3 tasks published (reserved)
  CNT_HEAD = 18,    // level-3 tasks taken
  CNT_PRODUCERS = 19,  // frontier entries fully walked (their tasks, if any, published)
  CNT_SPLIT = 20,   // level-3 sets handed out as tasks (stats)
  CNT_DBG_RUNS = 21,     // k_last4: x2 runs started (GCSM_TRACE)
  CNT_DBG_PINBYTES = 22, // k_last4: zero-copy bytes copied by run pins
  CNT_DBG_PINS = 23,     // k_last4: runs pinned
  CNT_CACHED = 24,       // GPU packer (query 0's block): cached vertices, cached bytes, internal error flag
  // fetch-once staging of zero-copy lists: bytes copied host -> batch arena, lists staged,
  // algorithmic bytes then served from the arena (HBM)
  CNT_STAGE_FILL = 27,
  CNT_STAGE_LISTS = 28,
  CNT_STAGE_HIT = 29,
  // B_comp (measurement mode only): bytes of the DISTINCT main lists the query's kernels touched,
  // by where they lived: HBM cache, pinned host (zero-copy), the batch's uploaded lists of U
  CNT_BCOMP = 30,
  CNT_PEER = 33,  // NVLink peer cache (NEXT-3): algorithmic list bytes read from a linked peer's HBM cache
  // k_extend work profile (GCSM_TRACE): entries walked, entries pruned by the hoisted last-level set, level-3 and
  // level-4 nodes, last-level driver elements
  CNT_X_ENTRIES = 34,
  CNT_X_PRUNED = 35,
  CNT_X_L3 = 36,
  CNT_X_L4 = 37,
  CNT_X_LAST = 38,
  CNT_X_L3F = 39,  // level-3 nodes kept by the level-3 filter
  CNT_WFILL = 40,  // the walks' fetch-once staging (query 0's block): bytes filled, lists, bytes served
  CNT_WLISTS = 41,
  CNT_WHIT = 42,
  CNT_WALG = 43,   // per query: algorithmic list bytes its walks read (driver scans + membership probes, §8d)
  CNT_WDBG = 44,   // per query, k_walks work profile (GCSM_TRACE): level-2 roots, lane-walked nodes, DFS descents, steps
  CNT_XT = 48,     // k_extend timing profile (cycles): sum and max of the warps' frontier phase, max warp, max entry,
                   // then the largest single-entry time of each phase (hoist, F, level-3 set, filter, rest)
  CNT_N = 57
};

struct MatchArgs {
  const DevPlan *plans;     // per-context query plans (2 per term)
  const VDesc *vdesc;
  const uint16_t *lab;      // nullptr if unlabelled
  const DRec *drec;
  const int32_t *dlist;
  const Unit *units;
  int64_t n_units;
  int2 *f2;                 // level-2 frontier: (candidate, unit index)
  int64_t f2_cap;
  int2 *useg;               // per unit: (offset, count) of its level-2 candidates in f2
  int32_t *scratch;         // per-warp stacks
  const int32_t *scratch_end;
  const int32_t *group;     // frontier entry indices grouped by candidate (nullptr: frontier order)
  int64_t scratch_stride;   // ints per warp
  int32_t dcap;             // ints per stack level (>= max list length)
  unsigned long long *cnt;  // CNT_N counters
  const char *cache_lo, *cache_hi;  // HBM cache address range (hit/miss accounting)
  const char *ubuf_lo, *ubuf_hi;    // the batch's uploaded stable lists of U (device-resident, delta accounting)
  const int32_t *sidx;              // sampled index of the host lists: every GCSM_SIDX_STRIDE-th element (nullptr: none)
  const uint32_t *soff;             // per vertex: offset of its samples in sidx, 0xffffffff = not indexed
  int32_t *tup_add;         // list mode: k ints per tuple
  uint64_t tup_add_cap;
  int32_t *tup_rem;
  uint64_t tup_rem_cap;
  int32_t k;
  int32_t n_plans;          // plans[] entries (2 m)
  int32_t listing;
  int32_t acc_base;         // CNT_ACC_L2 or CNT_ACC_EXT (set by the launchers)
  // level-3 work sharing (k >= 5): a warp whose level-3 candidate set is large copies it to the arena and
  // publishes slices of it as tasks that idle warps take (STMatch-style work sharing)
  int32_t *arena;
  uint64_t arena_cap;       // ints
  struct Task *tasks;
  int32_t *task_ready;
  uint32_t task_cap;
  int32_t fsplit;
  int32_t merge2;           // two-list materialising intersections by merge path when cheaper (GCSM_MERGE2=1; off:
                            // measured no faster, profiles/ab9_r02.txt)           // k >= 5: share large level-3 sets before the level-3 filter (GCSM_NO_FSPLIT=1: after)
  int32_t task_gen;         // ready-flag value of this launch (no per-launch clearing)
  // fetch-once staging of zero-copy lists within a batch: per vertex state word (epoch << 40 | ready << 39 |
  // offset), the batch arena and its bump counter; nullptr = off
  unsigned long long *stage_state;
  int32_t *stage_arena;
  unsigned long long stage_cap;  // ints
  unsigned long long *stage_bump;
  uint32_t stage_epoch;          // 24 bits, never 0
  uint32_t stage_min;            // shortest list (ints) routed through the arena
  int32_t stage_policy;          // shared-memory staging of device-resident probe lists: 0 bytes model, 1 latency
  int32_t filter3;               // level-3 filter on (LevelPlan::fmask)
  int32_t hoist;                 // hoisted last-level set on (LevelPlan::hmask)
  uint32_t *touched;             // B_comp measurement: bitmap of vertices whose main list was read (nullptr = off)
  // NVLink peer cache: the linked peers' descriptor arrays and cache address ranges of this
  // batch; a zero-copy miss whose list a peer holds in HBM is read from there (peer / NVLink) instead
  int32_t npeer;
  const VDesc *peer_vdesc[GCSM_MAX_PEERS];
  const char *peer_lo[GCSM_MAX_PEERS], *peer_hi[GCSM_MAX_PEERS];  // the peer's cache range (its addresses)
  const char *peer_map[GCSM_MAX_PEERS];  // where that range is mapped here (= peer_lo within one process)
};

struct Task {
  int64_t e;        // level-2 frontier entry (unit, x2)
  uint64_t off;     // its level-3 candidate set in the arena
  uint32_t n;       // set size
  uint32_t lo, hi;  // the slice of positions this task iterates
  uint32_t pad;
  uint64_t xoff;    // the entry's hoisted last-level set H then its level-3 filter set F, in the arena (computed once
                    // by the producer: a taker copies them instead of intersecting the entry's lists again)
  uint32_t hn, nF1, nF, pad2;
};
static_assert(sizeof(Task) == 56, "Task is read as 7 x 8 bytes");

// plans live in a per-context device buffer (contexts may run concurrently)
cudaError_t upload_plans(DevPlan *dst, const DevPlan *plans, int n, cudaStream_t s);
// grid sizes: persistent CTAs (multiple of the SM count)
int match_grid(int device, int *warps_total);
cudaError_t launch_level2(const MatchArgs &a, int grid, cudaStream_t s);
cudaError_t launch_extend(const MatchArgs &a, int grid, cudaStream_t s);
// counting sort of the level-2 frontier by candidate vertex (hist: n uint32; bsum: ceil(n/2048) uint32)
cudaError_t launch_group_frontier(const MatchArgs &a, int32_t n_vertices, uint32_t *hist, uint32_t *bsum,
                                  int32_t *group, cudaStream_t s);
cudaError_t launch_gather_lists(char *dst, const char *src, const uint64_t *tri, int64_t n, cudaStream_t s);
// B_comp (measurement mode): sum the main-list bytes of the vertices in the touched bitmap by where they live;
// out[0..2] += (HBM cache, pinned host, uploaded U lists)
cudaError_t launch_bcomp(const uint32_t *touched, int32_t n, const VDesc *vdesc, const char *cache_lo,
                         const char *cache_hi, const char *ubuf_lo, const char *ubuf_hi, unsigned long long *out,
                         cudaStream_t s);
cudaError_t launch_patch_vdesc(VDesc *vdesc, const int64_t *idx, const VDesc *val, int64_t n, cudaStream_t s);
// sampled-index updates: rec[i] = (vertex, offset, count, staging position); samples staged contiguously
cudaError_t launch_sidx_update(int32_t *sidx, uint32_t *soff, const int4 *rec, int64_t n, const int32_t *staged,
                               cudaStream_t s);

}  // namespace gcsm
