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

// Persistent per-batch scratch. Every node's read of a list is a record (vertex, level, B); records go to
// thread-local buffers partitioned by vertex range (kPartLog2 ids per partition), and each partition is then
// reduced by one thread in a cache-resident dense window: no scattered atomics into n-sized arrays, ids come
// out sorted, and the integer sums are identical to any other summation order.
struct EstRec {
  int32_t v;
  uint32_t level;
  uint64_t B;
};
struct EstimatorScratch {
  int32_t n = 0;
  int threads = 0;
  int parts = 0;
  std::vector<std::vector<EstRec>> buf;  // [thread * parts + partition]
};

struct EstimatorOutput {
  std::vector<int32_t> ids;      // ascending
  std::vector<uint64_t> levcnt;  // 8 per id: Σ B at levels 1..k-2
};

// skip sampling of children in BINV's domain (estimator.cpp; the device walker mirrors it bit for bit)
constexpr uint32_t kSkipSeg = 1024;   // driver elements per segment (= kEstItem, the level-1 work item)
constexpr int kSkipLog = 10;          // r0^(2^i), i = 0..10: gaps up to 2 kSkipSeg - 1
constexpr uint64_t kSkipTag = 0x53B1000000000000ULL;  // segment s's stream: rng_chain(node key, kSkipTag + s)
int64_t binom_pos(uint64_t ck, int64_t n, double p, double r0);  // Bin(n, p) | >= 1, n p < 10, r0 = (1-p)^n
void skip_table(double r0, double *pw);
uint32_t skip_gap(const double *pw, double u);
uint64_t skip_uniform_bits(uint64_t segkey, uint64_t j);

uint64_t walk_budget(uint64_t N1, uint64_t D, int k);
double stirling_small(int k);  // BTRD's Stirling correction for k < 10 (lgamma; the GPU sampler's table)
void run_estimator(const EstimatorInput &in, EstimatorScratch &scr, EstimatorOutput &out);
double estimate_value(const uint64_t *lev, int k, uint64_t N1, uint64_t D, uint64_t M);

}  // namespace gcsm
