// estimator.h — host-side random-walk estimator interface (step ②).
#pragma once
#include <functional>

#include "internal.h"

namespace gcsm {

// A view of one adjacency list on the host: two disjoint sorted segments.
struct HList {
  const int32_t *a;
  uint32_t na;
  const int32_t *b;
  uint32_t nb;
};

struct EstimatorInput {
  const DevPlan *plans;
  const Unit *units;
  int64_t n_units;
  uint64_t N1, D, M;
  uint64_t seed, batch_seq;
  const uint16_t *labels;  // nullptr = all 0
  int32_t n;               // vertex universe
  int threads;
  std::function<HList(int32_t, int)> view;  // (vertex, View) -> host list view
};

// Persistent dense accumulators (n x (k-2) sums + a touched bitmap), reset
// sparsely after each batch: O(records) accumulation, ids come out sorted.
struct EstimatorScratch {
  int32_t n = 0;
  int levels = 0;
  std::vector<uint64_t> sums;     // [levels][n]
  std::vector<uint64_t> touched;  // n bits
};

struct EstimatorOutput {
  std::vector<int32_t> ids;      // ascending
  std::vector<uint64_t> levcnt;  // 8 per id: Σ B at levels 1..k-2
};

uint64_t walk_budget(uint64_t N1, uint64_t D, int k);
void run_estimator(const EstimatorInput &in, EstimatorScratch &scr, EstimatorOutput &out);
double estimate_value(const uint64_t *lev, int k, uint64_t N1, uint64_t D, uint64_t M);

}  // namespace gcsm
