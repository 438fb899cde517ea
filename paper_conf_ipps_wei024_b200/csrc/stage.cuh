// stage.cuh — device helpers shared by the matching kernels (kernels.cu) and the GPU walks (estimator_gpu.cu):
// the warp-cooperative bulk list copy and the fetch-once staging of zero-copy lists within a batch
// (DESIGN.md §1d).
#pragma once
#include <cstdint>

namespace gcsm {

struct StageRef {
  unsigned long long *state;  // per vertex: epoch << 40 | ready << 39 | offset (ints)
  int32_t *arena;
  unsigned long long cap;     // ints
  unsigned long long *bump;
  uint32_t epoch;             // 24 bits, never 0
};

#ifdef __CUDACC__
namespace {
// Warp-cooperative bulk copy of a list (16-byte aligned source; lists are
// allocated in 16-byte granules so reading up to round4(n) ints stays inside
// the allocation). 4 x 16 B loads per lane are issued before any store, so a
// warp keeps 2 KB in flight: a zero-copy list crosses PCIe at link speed
// instead of one dependent 32 B sector per binary-search step.
__device__ __forceinline__ void warp_copy(int32_t *dst, const int32_t *src, uint32_t n, int lane) {
  __syncwarp();  // every lane is done reading what this buffer held before (WAR across lanes)
  const uint32_t n4 = (n + 3) >> 2;
  const int4 *s4 = reinterpret_cast<const int4 *>(src);
  int4 *d4 = reinterpret_cast<int4 *>(dst);
  for (uint32_t base = 0; base < n4; base += 128) {
    const uint32_t i0 = base + lane, i1 = i0 + 32, i2 = i0 + 64, i3 = i0 + 96;
    int4 v0, v1, v2, v3;
    if (i0 < n4) v0 = s4[i0];
    if (i1 < n4) v1 = s4[i1];
    if (i2 < n4) v2 = s4[i2];
    if (i3 < n4) v3 = s4[i3];
    if (i0 < n4) d4[i0] = v0;
    if (i1 < n4) d4[i1] = v1;
    if (i2 < n4) d4[i2] = v2;
    if (i3 < n4) d4[i3] = v3;
  }
}

#ifndef GCSM_STAGE_DEEP
#define GCSM_STAGE_DEEP 0
#endif
// The arena fill's copy (out of line, in stage_fetch): GCSM_STAGE_DEEP = 1 keeps 8 x 16 B per lane in flight (4 KB
// per warp) for hub lists crossing PCIe.
__device__ __forceinline__ void warp_copy_fill(int32_t *dst, const int32_t *src, uint32_t n, int lane) {
#if GCSM_STAGE_DEEP
  __syncwarp();
  const uint32_t n4 = (n + 3) >> 2;
  const int4 *s4 = reinterpret_cast<const int4 *>(src);
  int4 *d4 = reinterpret_cast<int4 *>(dst);
  for (uint32_t base = 0; base < n4; base += 256) {
    int4 v[8];
#pragma unroll
    for (int k = 0; k < 8; ++k)
      if (base + lane + 32 * k < n4) v[k] = s4[base + lane + 32 * k];
#pragma unroll
    for (int k = 0; k < 8; ++k)
      if (base + lane + 32 * k < n4) d4[base + lane + 32 * k] = v[k];
  }
#else
  warp_copy(dst, src, n, lane);
#endif
}

// ---- fetch-once staging of zero-copy lists within a batch -------------------------------------
// The first warp of the batch that needs vertex v's zero-copy main list claims it (CAS of its state word from an
// older epoch to "loading"), copies it over PCIe into the batch arena (bump-allocated, 128-byte granules so that
// no two lists share an L1 line) and publishes (epoch, ready, offset); every later read of that list in the batch,
// by any warp or any later kernel of the batch, is an HBM read. A warp that finds the list loading waits for it
// (the loader waits on nothing, so this cannot deadlock). Arena full: the list stays zero-copy ("no room").
// The arena holds the batch's MAIN lists (v not in U: base(v), unchanged during the batch); the next batch has a
// new epoch, so nothing stale is ever served.
constexpr unsigned long long kStReady = 1ull << 39, kStOff = (1ull << 39) - 1;

// the state word with acquire semantics (device scope): the arena copy published before it is visible after it
__device__ __forceinline__ unsigned long long stage_word(const unsigned long long *w) {
  unsigned long long v;
  asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(w) : "memory");
  return v;
}

// Outcome of a fetch-once lookup: where the list is read from and how (kStZc: zero-copy, no room this batch;
// kStServed: an arena copy made by someone else; kStFilled: this warp copied it). Returned by value so that the
// callers' byte counters stay in registers (a reference argument of an out-of-line call would pin them to local
// memory).
enum : uint32_t { kStZc = 0, kStServed = 1, kStFilled = 2 };
struct StageRes {
  const int32_t *p;
  uint32_t how;
};
__device__ __forceinline__ void stage_count(const StageRes &r, uint32_t ml, unsigned long long &sfill,
                                            unsigned long long &slists, unsigned long long &shit) {
  if (r.how == kStFilled) {
    sfill += 4ull * ml;
    slists += 1;
  } else if (r.how == kStServed) {
    shit += 4ull * ml;
  }
}
__device__ __noinline__ StageRes stage_fetch(const StageRef &A, int32_t v, const int32_t *hp, uint32_t ml, int lane) {
  const unsigned long long ep = (unsigned long long)A.epoch << 40;
  unsigned long long res = 0;
  int claimed = 0;
  if (lane == 0) {
    unsigned long long *w = A.state + v;
    unsigned long long cur = stage_word(w);
    unsigned ns = 32;
    for (;;) {
      if ((cur & ~((1ull << 40) - 1)) == ep) {  // this batch's: ready, no room, or being loaded
        if (cur & kStReady) {
          res = cur & kStOff;
          break;
        }
        __nanosleep(ns);
        if (ns < 2048) ns <<= 1;
        cur = stage_word(w);
        continue;
      }
      const unsigned long long prev = atomicCAS(w, cur, ep | kStOff);  // claim: loading
      if (prev == cur) {
        claimed = 1;
        break;
      }
      cur = prev;
    }
    if (claimed) {
      const unsigned long long n32 = ((unsigned long long)ml + 31) & ~31ull;
      const unsigned long long off = atomicAdd(A.bump, n32);
      if (off + n32 > A.cap) {
        atomicExch(w, ep | kStReady | kStOff);  // no room this batch: zero-copy for everyone
        claimed = 0;
        res = kStOff;
      } else {
        res = off;
      }
    }
  }
  claimed = __shfl_sync(0xffffffffu, claimed, 0);
  res = __shfl_sync(0xffffffffu, res, 0);
  if (claimed) {
    int32_t *dst = A.arena + res;
    warp_copy_fill(dst, hp, ml, lane);
    __syncwarp();
    __threadfence();  // release: the copy before the state word
    if (lane == 0) atomicExch(A.state + v, ep | kStReady | res);
    return StageRes{dst, kStFilled};
  }
  __syncwarp();
  if (res == kStOff) return StageRes{hp, kStZc};
  return StageRes{A.arena + res, kStServed};
}

}  // namespace
#endif  // __CUDACC__

}  // namespace gcsm
