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
  CNT_COPIED = 3,   // bytes bulk-copied from host memory by the kernels' staging (real zero-copy reads)
  // per kernel, 3 consecutive slots: list bytes (algorithmic: 4 B x list length per use) served from
  // the HBM cache, zero-copy from pinned host memory, and from the device delta segments (ins/del of U)
  CNT_ACC_L2 = 10,
  CNT_ACC_EXT = 13,
  CNT_N = 16
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
  int32_t *tup_add;         // list mode: k ints per tuple
  uint64_t tup_add_cap;
  int32_t *tup_rem;
  uint64_t tup_rem_cap;
  int32_t k;
  int32_t listing;
  int32_t acc_base;         // CNT_ACC_L2 or CNT_ACC_EXT (set by the launchers)
};

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
cudaError_t launch_patch_vdesc(VDesc *vdesc, const int64_t *idx, const VDesc *val, int64_t n, cudaStream_t s);

}  // namespace gcsm
