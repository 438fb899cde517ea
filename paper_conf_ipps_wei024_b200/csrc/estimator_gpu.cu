// estimator_gpu.cu — steps ② (random-walk access-frequency estimation, §IV) and ③ (cache ranking and
// packing) on sm_100a, enqueued on the context's stream before the matching kernels.
//
// ② k_walks: warp per level-1 node (a unit with its host-drawn B_1 ~ Bin(M, 1/N1)), DFS over the merged
//    walks of §IV-B inside the warp: a node at level l records B on every list its next position reads (eq. (3),
//    P:204; R17) into dense per-query integer sums; its children are the candidates of the next position (R18),
//    the lanes taking 32 consecutive driver elements, each child drawing B' ~ Bin(B, 1/D) from its own key
//    (R20, R22) and surviving if B' > 0 and it belongs to every other backward list. Integer atomics make the sums
//    independent of the visiting order, so they equal the host walker's and the oracle's bit for bit.
// ③ the touched vertices (a bitmap, compacted in id order) get their estimate (eq. (3) averaged over M, summed
//    over standing queries); the ranking cut of R23 (estimate desc, id asc, longest prefix under the budget) is
//    found without a sort: byte-weighted histograms over the score's IEEE bits, 12 bits per pass, narrow the cut
//    to one exact score value (positive doubles order like their bit patterns); the vertices strictly above it all
//    fit; the ties at it are taken in id order while they fit (an inclusive scan). The selected lists are copied
//    into this batch's cache buffer from where their descriptors point (the previous buffer: HBM -> HBM, else the
//    pinned host store over PCIe), then the descriptors are switched (previous selection back to host, new one to
//    its slot).
//
// Floating point: the binomial samplers and the score are transcribed from the host code with explicit
// round-to-nearest intrinsics (__dmul_rn, __dadd_rn, __dsub_rn, __ddiv_rn, __dsqrt_rn) so nvcc cannot contract
// them into FMAs: the same IEEE operation sequence gives the same doubles. BINV's r0 = (1-p)^n comes from a host
// table (glibc pow), BTRD's Stirling terms for k < 10 from a host table (glibc lgamma); BTRD's log is CUDA's
// (max 1 ulp; it decides only comparisons that are not within an ulp of a tie — DESIGN.md).

#include "estimator.h"
#include "estimator_gpu.cuh"

namespace gcsm {
namespace {

constexpr unsigned FULL = 0xffffffffu;

__device__ __forceinline__ unsigned long long dmix(unsigned long long z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}
__device__ __forceinline__ unsigned long long dchain(unsigned long long h, unsigned long long x) {
  return dmix(h + 0x9E3779B97F4A7C15ULL * (x + 1));
}

#define DM(a, b) __dmul_rn((a), (b))
#define DA(a, b) __dadd_rn((a), (b))
#define DS(a, b) __dsub_rn((a), (b))
#define DV(a, b) __ddiv_rn((a), (b))

struct DUni {
  unsigned long long key, j;
  __device__ __forceinline__ double next() {
    ++j;
    return DM((double)(dmix(key + 0xD1B54A32D192ED03ULL * j) >> 11), 1.0 / 9007199254740992.0);
  }
};

struct BinTab {
  double pD;
  const double *r0tab;
  int64_t r0n;
  const double *sfc;  // 10 entries
  int32_t *err;
};

__device__ __forceinline__ double d_sfc(const BinTab &T, int64_t k) {
  if (k < 10) return T.sfc[k];
  const double r = DV(1.0, (double)(k + 1)), r2 = DM(r, r);
  return DM(DS(1.0 / 12.0, DM(DS(1.0 / 360.0, DM(1.0 / 1260.0, r2)), r2)), r);
}

// BINV (n p < 10): estimator.cpp binv with r0 = (1-p)^n from the host table.
__device__ int64_t d_binv(DUni &U, int64_t n, double p, double r0) {
  const double q = DS(1.0, p);
  const double s = DV(p, q), a = DM((double)(n + 1), s);
  for (;;) {
    double r = r0, u = U.next();
    int64_t x = 0;
    while (u > r) {
      u = DS(u, r);
      x += 1;
      if (x > n) break;
      r = DM(r, DS(DV(a, (double)x), s));
    }
    if (x <= n) return x;
  }
}

// BTRD (n p >= 10): estimator.cpp btrd, operation for operation.
__device__ int64_t d_btrd(DUni &U, int64_t n, double p, const BinTab &T) {
  const double q = DS(1.0, p);
  const double m = floor(DM((double)(n + 1), p));
  const double r = DV(p, q), nr = DM((double)(n + 1), r), npq = DM(DM((double)n, p), q);
  const double spq = __dsqrt_rn(npq);
  const double b = DA(1.15, DM(2.53, spq));
  const double a = DA(DA(-0.0873, DM(0.0248, b)), DM(0.01, p));
  const double c = DA(DM((double)n, p), 0.5);
  const double alpha = DM(DA(2.83, DV(5.1, b)), spq);
  const double vr = DS(0.92, DV(4.2, b));
  const double urvr = DM(0.86, vr);
  const int64_t mi = (int64_t)m;
  for (;;) {
    double v = U.next(), u;
    if (v <= urvr) {
      u = DS(DV(v, vr), 0.43);
      return (int64_t)floor(DA(DM(DA(DV(DM(2.0, a), DS(0.5, fabs(u))), b), u), c));
    }
    if (v >= vr) {
      u = DS(U.next(), 0.5);
    } else {
      u = DS(DV(v, vr), 0.93);
      u = DS(u < 0 ? -0.5 : 0.5, u);
      v = DM(U.next(), vr);
    }
    const double us = DS(0.5, fabs(u));
    const double kd = floor(DA(DM(DA(DV(DM(2.0, a), us), b), u), c));
    if (kd < 0.0 || kd > (double)n) continue;
    const int64_t ki = (int64_t)kd;
    v = DV(DM(v, alpha), DA(DV(a, DM(us, us)), b));
    const int64_t km = ki > mi ? ki - mi : mi - ki;
    if (km <= 15) {
      double f = 1.0;
      if (mi < ki) {
        for (int64_t i = mi + 1; i <= ki; ++i) f = DM(f, DS(DV(nr, (double)i), r));
      } else if (mi > ki) {
        for (int64_t i = ki + 1; i <= mi; ++i) v = DM(v, DS(DV(nr, (double)i), r));
      }
      if (v <= f) return ki;
      continue;
    }
    v = log(v);
    const double kmd = (double)km;
    const double rho = DM(DV(kmd, npq), DA(DV(DA(DM(DA(DV(kmd, 3.0), 0.625), kmd), 1.0 / 6.0), npq), 0.5));
    const double t = DV(DM(-kmd, kmd), DM(2.0, npq));
    if (v < DS(t, rho)) return ki;
    if (v > DA(t, rho)) continue;
    const double nm = (double)(n - mi + 1);
    const double h = DA(DA(DM(DA(m, 0.5), log(DV(DA(m, 1.0), DM(r, nm)))), d_sfc(T, mi)), d_sfc(T, n - mi));
    const double nk = (double)(n - ki + 1);
    const double rhs = DS(DS(DA(DA(h, DM((double)(n + 1), log(DV(nm, nk)))),
                                DM(DA(kd, 0.5), log(DV(DM(nk, r), DA(kd, 1.0))))),
                             d_sfc(T, ki)),
                          d_sfc(T, n - ki));
    if (v <= rhs) return ki;
  }
}

// estimator.cpp binomial(key, n, p) for p = 1/D.
__device__ __forceinline__ int64_t d_binomial(unsigned long long key, int64_t n, const BinTab &T) {
  const double p = T.pD;
  if (n <= 0 || p <= 0.0) return 0;
  if (p >= 1.0) return n;
  DUni U{key, 0};
  if (p > 0.5) {  // unreachable: p = 1/D with an integer D >= 2
    atomicExch(T.err, 1);
    return 0;
  }
  if (DM((double)n, p) < 10.0) {
    if (n >= T.r0n) {
      atomicExch(T.err, 2);
      return 0;
    }
    return d_binv(U, n, p, T.r0tab[n]);
  }
  return d_btrd(U, n, p, T);
}

__device__ __noinline__ int64_t d_binomial_ool(unsigned long long key, int64_t n, BinTab T) { return d_binomial(key, n, T); }

// ---- skip sampling (estimator.cpp skip_table / skip_gap / binom_pos, operation for operation) ------------------
static_assert(kSkipSeg == (uint32_t)kEstItem, "a level-1 work item is one skip segment");
__device__ __forceinline__ void d_skip_table(double r0, double *pw) {
  pw[0] = r0;
#pragma unroll
  for (int i = 1; i < kSkipLog + 1; ++i) pw[i] = DM(pw[i - 1], pw[i - 1]);
}
__device__ __forceinline__ uint32_t d_skip_gap(const double *pw, double u) {
  double cur = 1.0;
  uint32_t g = 0;
#pragma unroll
  for (int i = kSkipLog; i >= 0; --i) {
    const double c = DM(cur, pw[i]);
    if (c >= u) {
      cur = c;
      g += 1u << i;
    }
  }
  return g;
}
__device__ __noinline__ int64_t d_binom_pos(unsigned long long ck, int64_t n, double p, double r0) {
  DUni U{ck, 0};
  const double q = DS(1.0, p);
  const double s = DV(p, q), a = DM((double)(n + 1), s);
  for (;;) {
    double u = DA(r0, DM(DS(1.0, r0), U.next()));
    double r = r0;
    int64_t x = 0;
    while (u > r) {
      u = DS(u, r);
      x += 1;
      if (x > n) break;
      r = DM(r, DS(DV(a, (double)x), s));
    }
    if (x > n) continue;
    return x < 1 ? 1 : x;
  }
}
__device__ __forceinline__ double d_skip_uniform(unsigned long long segkey, unsigned long long j) {
  return DM((double)(dmix(segkey + 0xD1B54A32D192ED03ULL * j) >> 11), 1.0 / 9007199254740992.0);
}
// inclusive warp scan of (g + 1): the driver offset (from the step's start) just past each lane's selection
__device__ __forceinline__ uint32_t skip_scan(uint32_t g, int lane) {
  uint32_t x = g + 1;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t y = __shfl_up_sync(FULL, x, o);
    if (lane >= o) x += y;
  }
  return x;
}

struct LR {
  const int32_t *m;
  uint32_t ml;
  const int32_t *x;
  uint32_t xl;
};

__device__ __forceinline__ LR view_of(const VDesc *vdesc, const DRec *drec, const int32_t *dlist, int32_t v, int vw) {
  const int4 raw = __ldg(reinterpret_cast<const int4 *>(vdesc + v));
  LR r;
  r.m = reinterpret_cast<const int32_t *>((unsigned long long)(unsigned)raw.x | ((unsigned long long)(unsigned)raw.y << 32));
  r.ml = (uint32_t)raw.z;
  r.x = nullptr;
  r.xl = 0;
  const uint32_t upd = (uint32_t)raw.w;
  if (upd != 0 && vw != VIEW_S) {
    const int4 e = __ldg(reinterpret_cast<const int4 *>(drec + (upd - 1)));
    if (vw == VIEW_NEW) {
      r.x = dlist + e.x;
      r.xl = (uint32_t)e.y;
    } else {
      r.x = dlist + e.z;
      r.xl = (uint32_t)e.w;
    }
  }
  return r;
}

__device__ __forceinline__ bool has(const int32_t *a, uint32_t n, int32_t v) {
  uint32_t lo = 0, hi = n;
  while (lo < hi) {
    const uint32_t mid = (lo + hi) >> 1;
    const int32_t x = a[mid];
    if (x < v) lo = mid + 1;
    else hi = mid;
  }
  return lo < n && a[lo] == v;
}

// One record of eq. (3)'s sums: B more reads of vertex w's list at tree level index li (R17). The touched bit is
// checked through L2 first: the seed vertices of a unit are touched by every node below it, and an atomic to an
// already-set word is a serialised round trip for nothing.
__device__ __forceinline__ void rec(unsigned long long *levcnt, int levels, uint32_t *touched, int32_t w, int li,
                                    unsigned long long B) {
  atomicAdd(levcnt + (size_t)w * levels + li, B);
  const uint32_t bit = 1u << (w & 31);
  if (!(__ldcg(touched + (w >> 5)) & bit)) atomicOr(touched + (w >> 5), bit);
}

struct WalkArgs {
  const DevPlan *plans;
  const EstUnit *units;
  int64_t n_units;
  const int2 *items;
  int64_t n_items;
  EstNode2 *f2;
  int64_t f2_cap;
  unsigned long long *f2_count;
  unsigned long long *cursor2;
  unsigned long long *levcnt;
  int32_t levels;
  const VDesc *vdesc;
  const DRec *drec;
  const int32_t *dlist;
  const uint16_t *lab;
  uint32_t *touched;
  unsigned long long *cursor;
  BinTab T;
  StageRef stage;            // fetch-once staging (stage.state == nullptr: off)
  unsigned long long *alg_cnt;  // algorithmic list bytes read (or nullptr)
  int32_t walk_stage;           // skip-sampled drivers: 0 always staged, 1 when >= 1 selection is expected, 2 never
  uint32_t stage_min;
  unsigned long long *stage_cnt;
  const char *dev_lo[2], *dev_hi[2];
  const int32_t *sidx;          // sampled index of the host lists (nullptr: plain binary searches)
  const uint32_t *soff;
  int32_t lane_leaf;            // level k-3 nodes one per lane (walk_leaf_parent; GCSM_WALK_LANE=0: warp-wide DFS)
};

// Membership of v in vertex w's main list m[0..ml): a list in the pinned host store is probed through its sampled
// index in HBM (every 32nd element): a binary search over the samples, then ONE read of the 32-element
// window that can hold v (8 x 16 B in flight) instead of log2(ml) dependent round trips over PCIe. Lists in device
// memory (cache, the batch's U lists, the staging arena) are binary-searched in place.
__device__ __forceinline__ bool probe(const WalkArgs &A, int32_t w, const int32_t *m, uint32_t ml, int32_t v) {
  const char *pc = reinterpret_cast<const char *>(m);
  const bool dev = (pc >= A.dev_lo[0] && pc < A.dev_hi[0]) || (pc >= A.dev_lo[1] && pc < A.dev_hi[1]) ||
                   (A.stage.arena && m >= A.stage.arena && m < A.stage.arena + A.stage.cap);
  if (dev || !A.sidx || ml < 64) return has(m, ml, v);
  const uint32_t off = __ldg(A.soff + w);
  if (off == 0xffffffffu) return has(m, ml, v);
  const int32_t *smp = A.sidx + off;
  uint32_t lo = 0, hi = (ml + 31) >> 5;  // first sample > v
  while (lo < hi) {
    const uint32_t mid = (lo + hi) >> 1;
    if (__ldg(smp + mid) <= v) lo = mid + 1;
    else hi = mid;
  }
  if (lo == 0) return false;  // v < m[0]
  const uint32_t base = 32u * (lo - 1), cnt = min(32u, ml - base);
  const int4 *p4 = reinterpret_cast<const int4 *>(m + base);  // lists are 16-byte aligned, 32-element windows too
  int4 q[8];
#pragma unroll
  for (int i = 0; i < 8; ++i) q[i] = 4 * i < (int)cnt ? p4[i] : make_int4(INT_MIN, INT_MIN, INT_MIN, INT_MIN);
  bool hit = false;
#pragma unroll
  for (int i = 0; i < 8; ++i)
    hit |= (4 * i + 0 < (int)cnt && q[i].x == v) | (4 * i + 1 < (int)cnt && q[i].y == v) |
           (4 * i + 2 < (int)cnt && q[i].z == v) | (4 * i + 3 < (int)cnt && q[i].w == v);
  return hit;
}

constexpr int kEW = 8;  // warps per block
struct EstLv {
  int32_t pos, ns, si, drv;
  unsigned long long B, key;
  unsigned long long T53;  // 1: the node samples its children by skip sampling (BINV's domain), ~0: one draw each
  unsigned long long uj;   // skip sampling: uniforms consumed in the current segment
  double r0;               // (1 - 1/D)^B (host table)
  double pw[kSkipLog + 1]; // r0^(2^i)
  const int32_t *dm, *dx;  // the node's driver list (main, delta segment), fixed at node entry
  uint32_t dml, dxl;
  const int32_t *pm[7];    // every backward main list as read (staged copy when zero-copy and staging is on)
  int32_t sv[32];
  unsigned long long sB[32], skey[32];
};
struct EstW {
  int32_t f[GCSM_MAXK];
  EstLv lv[GCSM_MAXK - 3];  // index = tree level - 2 (levels 2..k-2)
};

// Level 1 (phase A): warp per work item (a unit and kEstItem of its driver elements). The item at index 0 records
// the level-1 node's reads; children with B' > 0 are recorded directly when they are the last sampled level (k = 4)
// or appended to the level-2 node list (k >= 5) for k_walks.
__global__ void __launch_bounds__(kEW * 32) k_walks_l1(const __grid_constant__ WalkArgs A) {
  const BinTab T = A.T;
  const int lane = threadIdx.x & 31;
  for (;;) {
    unsigned long long it = 0;
    if (lane == 0) it = atomicAdd(A.cursor, 1ull);
    it = __shfl_sync(FULL, it, 0);
    if (it >= (unsigned long long)A.n_items) return;
    const int2 item = A.items[it];
    const EstUnit U = A.units[item.x];
    const DevPlan *P = A.plans + U.plan;
    const int k = P->k;
    const LevelPlan &Lp = P->lv[2];
    const int nb = Lp.nb;
    const int32_t f01[2] = {U.a, U.b};
    if (item.y == 0 && lane < nb) {
      const int32_t v = f01[Lp.bpos[lane]];
      rec(A.levcnt, A.levels, A.touched, v, 0, U.B);
    }
    if (k <= 3) continue;  // level 1 is the last sampled level
    LR L[7];
    int drv = 0;
    uint32_t best = 0xffffffffu;
    for (int b = 0; b < nb; ++b) {
      L[b] = view_of(A.vdesc, A.drec, A.dlist, f01[Lp.bpos[b]], Lp.bview[b]);
      const uint32_t t = L[b].ml + L[b].xl;
      if (t < best) {
        best = t;
        drv = b;
      }
    }
    const uint32_t end = min(best, (uint32_t)item.y + (uint32_t)kEstItem);
    const LevelPlan &L3 = P->lv[3];
    // emit one step's children: (k = 4) the reads of the level-2 nodes, (k >= 5) level-2 walk nodes
    // emit one step's children (level-2 nodes): the reads they share (position 3's lists at the seeds, positions 0
    // and 1) are recorded once per step with the children's summed B; (k = 4) each child records its own list
    // (position 2), (k >= 5) the child becomes a root of k_walks, which records that one
    auto emit = [&](bool ok, int32_t v, unsigned long long Bc, unsigned long long ck) {
      unsigned long long sumB = ok ? Bc : 0ull;
#pragma unroll
      for (int o = 16; o; o >>= 1) sumB += __shfl_xor_sync(FULL, sumB, o);
      if (sumB && lane < L3.nb && L3.bpos[lane] < 2) rec(A.levcnt, A.levels, A.touched, L3.bpos[lane] ? U.b : U.a, 1, sumB);
      if (k == 4) {
        if (ok)
          for (int b = 0; b < L3.nb; ++b)
            if (L3.bpos[b] == 2) rec(A.levcnt, A.levels, A.touched, v, 1, Bc);
      } else {
        const unsigned mask = __ballot_sync(FULL, ok);
        unsigned long long base = 0;
        if (lane == 0 && mask) base = atomicAdd(A.f2_count, (unsigned long long)__popc(mask));
        base = __shfl_sync(FULL, base, 0);
        if (ok) {
          const unsigned long long slot = base + __popc(mask & ((1u << lane) - 1u));
          if (slot < (unsigned long long)A.f2_cap) A.f2[slot] = EstNode2{U.a, U.b, v, U.plan, Bc, ck};
          else atomicExch(A.T.err, 3);
        }
      }
    };
    if ((int64_t)U.B < T.r0n && DM((double)U.B, T.pD) < 10.0) {  // BINV's domain: skip sampling of the item
      const double r0 = T.r0tab[U.B];
      double pw[kSkipLog + 1];
      d_skip_table(r0, pw);
      const unsigned long long segkey = dchain(U.key, kSkipTag + (unsigned long long)item.y / kSkipSeg);
      uint32_t pos = (uint32_t)item.y;
      unsigned long long uj = 0;
      while (pos < end) {
        const uint32_t g = d_skip_gap(pw, d_skip_uniform(segkey, uj + lane + 1));
        const uint32_t sel = pos + skip_scan(g, lane) - 1;
        const bool valid = sel < end;  // a prefix of the lanes
        const int nv = __popc(__ballot_sync(FULL, valid));
        bool ok = valid;
        int32_t v = 0;
        unsigned long long Bc = 0, ck = 0;
        if (ok) {
          v = sel < L[drv].ml ? L[drv].m[sel] : L[drv].x[sel - L[drv].ml];
          ok = v != U.a && v != U.b;
          if (ok && Lp.label >= 0) ok = (A.lab ? (int32_t)A.lab[v] : 0) == Lp.label;
          if (ok)
            for (int b = 0; b < nb; ++b)
              if (b != drv && !(has(L[b].m, L[b].ml, v) || (L[b].xl && has(L[b].x, L[b].xl, v)))) {
                ok = false;
                break;
              }
          if (ok) {
            ck = dchain(U.key, (unsigned long long)(uint32_t)v);
            Bc = (unsigned long long)d_binom_pos(ck, (int64_t)U.B, T.pD, r0);
          }
        }
        emit(ok, v, Bc, ck);
        if (nv < 32) break;
        pos = __shfl_sync(FULL, sel, 31) + 1;
        uj += 32;
      }
      continue;
    }
    for (uint32_t pos = (uint32_t)item.y; pos < end; pos += 32) {
      const uint32_t idx = pos + lane;
      bool ok = false;
      int32_t v = 0;
      unsigned long long Bc = 0, ck = 0;
      if (idx < end) {
        v = idx < L[drv].ml ? L[drv].m[idx] : L[drv].x[idx - L[drv].ml];
        ok = v != U.a && v != U.b;
        if (ok && Lp.label >= 0) ok = (A.lab ? (int32_t)A.lab[v] : 0) == Lp.label;
        if (ok) {
          ck = dchain(U.key, (unsigned long long)(uint32_t)v);
          const int64_t bc = d_binomial(ck, (int64_t)U.B, T);
          Bc = (unsigned long long)bc;
          ok = bc > 0;
        }
        if (ok)
          for (int b = 0; b < nb; ++b)
            if (b != drv && !(has(L[b].m, L[b].ml, v) || (L[b].xl && has(L[b].x, L[b].xl, v)))) {
              ok = false;
              break;
            }
      }
      emit(ok, v, Bc, ck);  // the child is a level-2 node (k = 4: of the last sampled level)
    }
  }
}

// A node at level k-3 whose B is in BINV's domain (its expected selections B x len / D are few; C4 prism6: the
// level-3 nodes) walked by ONE lane: it records B on its next position's backward lists, draws its children by the
// same skip sampling as the warp-wide step (one segment's gaps drawn one after another with uniforms j = 1, 2, ...
// of the segment's stream: the same draws), and every surviving child (level k-2, whose children are leaves)
// records its B' ~ Bin(B, 1/D) conditioned on >= 1 (d_binom_pos, the child's own key). Integer atomics: the sums
// equal the warp-wide DFS's bit for bit. f[0..cl-1] are the matched positions, v the node's vertex at cl.
struct WalkBytes {
  unsigned long long alg, hit;  // algorithmic list bytes read, bytes served by the staging arena
};
__device__ __noinline__ WalkBytes walk_leaf_parent(const WalkArgs &A, const DevPlan *P, const int32_t *f, int cl,
                                                   int32_t v, unsigned long long B, unsigned long long key) {
  unsigned long long walg = 0, whit = 0;
  const LevelPlan &Lq = P->lv[cl + 1];
  const int nb = Lq.nb;
  auto fat = [&](int p) { return p == cl ? v : f[p]; };
  for (int b = 0; b < nb; ++b)  // its own list (the shared ones at positions < cl: the parent's step)
    if (Lq.bpos[b] == cl) rec(A.levcnt, A.levels, A.touched, v, cl - 1, B);
  int drv = 0;
  LR D;
  uint32_t best = 0xffffffffu;
  for (int b = 0; b < nb; ++b) {
    const LR L = view_of(A.vdesc, A.drec, A.dlist, fat(Lq.bpos[b]), Lq.bview[b]);
    if (L.ml + L.xl < best) {
      best = L.ml + L.xl;
      drv = b;
      D = L;
    }
  }
  if (best == 0) return WalkBytes{walg, whit};
  // staged copies (this batch's arena) of the main lists, where another reader already fetched them
  auto staged = [&](int32_t vb, const int32_t *m, uint32_t ml) -> const int32_t * {
    if (!A.stage.state || ml < A.stage_min) return m;
    const unsigned long long st = stage_word(A.stage.state + vb);
    if ((st >> 40) == A.stage.epoch && (st & kStReady) && (st & kStOff) != kStOff) {
      whit += 4ull * ml;
      return A.stage.arena + (st & kStOff);
    }
    return m;
  };
  const int32_t *dm = staged(fat(Lq.bpos[drv]), D.m, D.ml);
  const double r0 = A.T.r0tab[B];
  double pw[kSkipLog + 1];
  d_skip_table(r0, pw);
  const LevelPlan &Lc = P->lv[cl + 2];  // the children's next position (they record, R17)
  unsigned long long sumB = 0;
  for (uint32_t s0 = 0; s0 < best; s0 += kSkipSeg) {
    const uint32_t s1 = min(best, s0 + kSkipSeg);
    const unsigned long long segkey = dchain(key, kSkipTag + s0 / kSkipSeg);
    uint32_t pos = s0;
    for (unsigned long long j = 1;; ++j) {
      const uint32_t sel = pos + d_skip_gap(pw, d_skip_uniform(segkey, j));
      if (sel >= s1) break;
      pos = sel + 1;
      walg += 4;
      const int32_t c = sel < D.ml ? dm[sel] : D.x[sel - D.ml];
      bool ok = c != v;
      for (int s2 = 0; s2 < cl && ok; ++s2) ok = f[s2] != c;
      if (ok && Lq.label >= 0) ok = (A.lab ? (int32_t)A.lab[c] : 0) == Lq.label;
      for (int b = 0; b < nb && ok; ++b) {
        if (b == drv) continue;
        const int32_t vb = fat(Lq.bpos[b]);
        const LR Lb = view_of(A.vdesc, A.drec, A.dlist, vb, Lq.bview[b]);
        walg += 4ull * (Lb.ml + Lb.xl);
        ok = probe(A, vb, staged(vb, Lb.m, Lb.ml), Lb.ml, c) || (Lb.xl && has(Lb.x, Lb.xl, c));
      }
      if (!ok) continue;
      const unsigned long long ck = dchain(key, (unsigned long long)(uint32_t)c);
      const unsigned long long Bc = (unsigned long long)d_binom_pos(ck, (int64_t)B, A.T.pD, r0);
      sumB += Bc;
      for (int b = 0; b < Lc.nb; ++b)
        if (Lc.bpos[b] == cl + 1) rec(A.levcnt, A.levels, A.touched, c, cl, Bc);
    }
  }
  if (sumB)  // the children's shared reads (positions <= cl), once
    for (int b = 0; b < Lc.nb; ++b)
      if (Lc.bpos[b] <= cl) rec(A.levcnt, A.levels, A.touched, fat(Lc.bpos[b]), cl, sumB);
  return WalkBytes{walg, whit};
}

// A step's children (level l+1 nodes, B summed over the warp in sb) read the lists of position l+2 at positions
// <= l together: one record per list for all of them (their own list, position l+1, each child records itself).
__device__ __forceinline__ void rec_shared(const WalkArgs &A, const DevPlan *P, const int32_t *f, int l,
                                           unsigned long long sb, int lane) {
#pragma unroll
  for (int o = 16; o; o >>= 1) sb += __shfl_xor_sync(FULL, sb, o);
  if (!sb) return;
  const LevelPlan &Lc = P->lv[l + 2];
  if (lane < Lc.nb && Lc.bpos[lane] <= l) rec(A.levcnt, A.levels, A.touched, f[Lc.bpos[lane]], l, sb);
}

// Levels >= 2 (phase B, k >= 5): warp per level-2 node, DFS over the rest of its subtree.
#ifndef GCSM_WALK_MINBLOCKS
#define GCSM_WALK_MINBLOCKS 3  // resident 256-thread blocks per SM for k_walks (latency hiding of its list reads)
#endif
__global__ void __launch_bounds__(kEW * 32, GCSM_WALK_MINBLOCKS) k_walks(const __grid_constant__ WalkArgs A) {
  __shared__ EstW sw[kEW];
  const BinTab T = A.T;
  const int lane = threadIdx.x & 31;
  EstW &W = sw[threadIdx.x >> 5];
  const unsigned long long n2 = min(*(volatile unsigned long long *)A.f2_count, (unsigned long long)A.f2_cap);
  unsigned long long wfill = 0, wlists = 0, whit = 0;  // fetch-once staging counters
  unsigned long long walg = 0;                         // algorithmic list bytes (driver scans + probes)
  unsigned long long d_root = 0, d_lane = 0, d_desc = 0, d_step = 0;  // work profile (CNT_WDBG)
  for (;;) {
    unsigned long long u = 0;
    if (lane == 0) u = atomicAdd(A.cursor2, 1ull);
    u = __shfl_sync(FULL, u, 0);
    if (u >= n2) {
      if (lane == 0 && A.alg_cnt) {
        atomicAdd(A.alg_cnt + 1, d_root);
        atomicAdd(A.alg_cnt + 2, d_lane);
        atomicAdd(A.alg_cnt + 3, d_desc);
        atomicAdd(A.alg_cnt + 4, d_step);
      }
      if (lane == 0 && A.stage_cnt && (wfill | wlists | whit)) {
        atomicAdd(A.stage_cnt + 0, wfill);
        atomicAdd(A.stage_cnt + 1, wlists);
        atomicAdd(A.stage_cnt + 2, whit);
      }
      if (lane == 0 && A.alg_cnt && walg) atomicAdd(A.alg_cnt, walg);
      return;
    }
    const EstNode2 N = A.f2[u];
    const DevPlan *P = A.plans + N.plan;
    const int k = P->k;
    ++d_root;
    __syncwarp();
    if (lane == 0) {
      W.f[0] = N.f0;
      W.f[1] = N.f1;
      W.f[2] = N.f2;
      W.lv[0].B = N.B;
      W.lv[0].key = N.key;
    }
    __syncwarp();
    int level = 2;
    bool fresh = true;
    while (level >= 2) {
      EstLv &S = W.lv[level - 2];
      const LevelPlan &Lp = P->lv[level + 1];
      const int nb = Lp.nb;
      if (fresh) {  // a node at `level` (positions 0..level matched) reads its next position's backward lists
        fresh = false;
        if (lane < nb && Lp.bpos[lane] == level)  // the lists at positions < level: recorded by the parent's step
          rec(A.levcnt, A.levels, A.touched, W.f[level], level - 1, S.B);
        if (level == k - 2) {  // its children are leaves: they read nothing (R17)
          --level;
          __syncwarp();
          continue;
        }
        // the node's driver (smallest backward list) and its BINV shortcut are fixed for all of its chunks
        LR L[7];
        int drv = 0;
        uint32_t best = 0xffffffffu;
        for (int b = 0; b < nb; ++b) {
          L[b] = view_of(A.vdesc, A.drec, A.dlist, W.f[Lp.bpos[b]], Lp.bview[b]);
          const uint32_t t = L[b].ml + L[b].xl;
          if (t < best) {
            best = t;
            drv = b;
          }
        }
        const int64_t Bn0 = (int64_t)S.B;
        const bool fast0 = Bn0 > 0 && T.pD > 0.0 && T.pD <= 0.5 && DM((double)Bn0, T.pD) < 10.0 && Bn0 < T.r0n;
        // zero-copy lists: the driver is fetched once per batch into HBM (under skip sampling only the selected
        // elements are read, but the staged copy serves every later reader); a probed list (only for the children
        // drawn) uses the staged copy when one exists, else a few in-place reads
        // staged unless the node expects less than one selection ((1 - r0) x length < 1: C4's level-3 nodes, whose
        // drivers would be fetched for nothing); reading every skip-sampled driver in place was measured slower
        // (31.4 K -> 22.6 K updated edges/s on C4: scattered PCIe reads, and probes of lists no driver staged)
        const bool stage_drv = !fast0 || A.walk_stage == 0 ||
                               (A.walk_stage == 1 && DM(DS(1.0, T.r0tab[Bn0]), (double)(L[drv].ml + L[drv].xl)) >= 1.0);
        for (int b = 0; b < nb; ++b) {
          const char *pc = reinterpret_cast<const char *>(L[b].m);
          if (!A.stage.state || L[b].ml < A.stage_min || (pc >= A.dev_lo[0] && pc < A.dev_hi[0]) ||
              (pc >= A.dev_lo[1] && pc < A.dev_hi[1]))
            continue;
          const int32_t vb = W.f[Lp.bpos[b]];
          if (b == drv && stage_drv) {
            const StageRes r = stage_fetch(A.stage, vb, L[b].m, L[b].ml, lane);
            stage_count(r, L[b].ml, wfill, wlists, whit);
            L[b].m = r.p;
          } else {
            const unsigned long long st = stage_word(A.stage.state + vb);
            if ((st >> 40) == A.stage.epoch && (st & kStReady) && (st & kStOff) != kStOff) {
              L[b].m = A.stage.arena + (st & kStOff);
              whit += 4ull * L[b].ml;
            }
          }
        }
        if (lane == 0)
          for (int b = 0; b < nb; ++b) S.pm[b] = L[b].m;
        walg += fast0 ? 0ull : 4ull * (L[drv].ml + L[drv].xl);  // a driver scanned whole (skip sampling: per selection)
        const int64_t Bn = (int64_t)S.B;
        const double pD = T.pD;
        const bool fast = Bn > 0 && pD > 0.0 && pD <= 0.5 && DM((double)Bn, pD) < 10.0 && Bn < T.r0n;
        if (lane == 0) {
          S.pos = 0;
          S.ns = 0;
          S.si = 0;
          S.drv = drv;
          S.dm = L[drv].m;
          S.dml = L[drv].ml;
          S.dx = L[drv].x;
          S.dxl = L[drv].xl;
          S.T53 = fast ? 1ull : ~0ull;
          S.uj = 0;
          if (fast) {
            S.r0 = T.r0tab[Bn];
            d_skip_table(S.r0, S.pw);
          }
        }
        __syncwarp();
        continue;
      }
      const int si = S.si, ns = S.ns;
      if (si == 0 && ns > 0 && level + 1 == k - 3 && A.lane_leaf) {
        // children at level k-3 in BINV's domain: one lane each (walk_leaf_parent) instead of one warp-wide DFS
        // descent per child
        bool fast = true;
        unsigned long long cB = 0, cK = 0;
        int32_t cv = 0;
        if (lane < ns) {
          cB = S.sB[lane];
          cK = S.skey[lane];
          cv = S.sv[lane];
          fast = cB > 0 && T.pD > 0.0 && T.pD <= 0.5 && DM((double)cB, T.pD) < 10.0 && (int64_t)cB < T.r0n;
        }
        if (__all_sync(FULL, fast)) {
          d_lane += ns;
          if (lane < ns) {
            const WalkBytes wb = walk_leaf_parent(A, P, W.f, level + 1, cv, cB, cK);
            walg += wb.alg;
            whit += wb.hit;
          }
          __syncwarp();
          if (lane == 0) S.si = ns;
          __syncwarp();
          continue;
        }
      }
      if (si < ns) {  // descend into the next surviving child
        ++d_desc;
        __syncwarp();
        if (lane == 0) {
          S.si = si + 1;
          W.f[level + 1] = S.sv[si];
          W.lv[level - 1].B = S.sB[si];
          W.lv[level - 1].key = S.skey[si];
        }
        __syncwarp();
        ++level;
        fresh = true;
        continue;
      }
      // the next (up to) 4 chunks of 32 driver elements: 4 loads per lane in flight, the BINV first-uniform test
      // (B' = 0 exactly when it fails, as in the host walker's pre-filter) inline, full draws out of line
      const uint32_t dml = S.dml, best = dml + S.dxl;
      const uint32_t pos = (uint32_t)S.pos;
      if (pos >= best) {
        __syncwarp();
        --level;
        continue;
      }
      const int p = level + 1;
      ++d_step;
      const int32_t *dm = S.dm, *dx = S.dx;
      const unsigned long long key = S.key, t53 = S.T53;
      const int64_t Bn = (int64_t)S.B;
      if (t53 != ~0ull) {  // skip sampling: one step of up to 32 selections in the current segment
        const uint32_t s1 = min(best, (pos / kSkipSeg + 1) * kSkipSeg);
        const unsigned long long segkey = dchain(key, kSkipTag + pos / kSkipSeg);
        const uint32_t g = d_skip_gap(S.pw, d_skip_uniform(segkey, S.uj + lane + 1));
        const uint32_t sel = pos + skip_scan(g, lane) - 1;
        const bool valid = sel < s1;  // a prefix of the lanes
        const int nv = __popc(__ballot_sync(FULL, valid));
        const uint32_t last = __shfl_sync(FULL, sel, 31);
        bool ok = valid;
        int32_t v = 0;
        walg += 4ull * (uint32_t)nv;  // the selected driver elements
        if (ok) {
          v = sel < dml ? dm[sel] : dx[sel - dml];
          for (int s2 = 0; s2 < p; ++s2) ok = ok && W.f[s2] != v;
          if (ok && Lp.label >= 0) ok = (A.lab ? (int32_t)A.lab[v] : 0) == Lp.label;
        }
        if (__any_sync(FULL, ok)) {  // membership in the other backward lists
          const int drv = S.drv;
          for (int b = 0; b < nb; ++b) {
            if (b == drv) continue;
            const LR Lb = view_of(A.vdesc, A.drec, A.dlist, W.f[Lp.bpos[b]], Lp.bview[b]);
            const int32_t *bm = S.pm[b];
            walg += 4ull * (Lb.ml + Lb.xl);
            if (ok) ok = probe(A, W.f[Lp.bpos[b]], bm, Lb.ml, v) || (Lb.xl && has(Lb.x, Lb.xl, v));
          }
        }
        unsigned long long Bc = 0, ck = 0;
        if (ok) {
          ck = dchain(key, (unsigned long long)(uint32_t)v);
          Bc = (unsigned long long)d_binom_pos(ck, Bn, T.pD, S.r0);
        }
        const unsigned msk = __ballot_sync(FULL, ok);
        __syncwarp();
        if (ok) {
          const int r = __popc(msk & ((1u << lane) - 1u));
          S.sv[r] = v;
          S.sB[r] = Bc;
          S.skey[r] = ck;
        }
        rec_shared(A, P, W.f, level, ok ? Bc : 0ull, lane);
        if (lane == 0) {
          S.ns = __popc(msk);
          S.si = 0;
          if (nv == 32 && last + 1 < s1) {
            S.pos = (int32_t)(last + 1);
            S.uj += 32;
          } else {  // the segment is done: the next one starts with a fresh stream
            S.pos = (int32_t)s1;
            S.uj = 0;
          }
        }
        __syncwarp();
        continue;
      }
      int32_t v[4];
      bool ok[4];
      unsigned long long Bc[4], ck[4];
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const uint32_t idx = pos + 32 * j + lane;
        ok[j] = idx < best;
        v[j] = ok[j] ? (idx < dml ? dm[idx] : dx[idx - dml]) : 0;
      }
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        for (int s2 = 0; s2 < p; ++s2) ok[j] = ok[j] && W.f[s2] != v[j];
        if (ok[j] && Lp.label >= 0) ok[j] = (A.lab ? (int32_t)A.lab[v[j]] : 0) == Lp.label;
        Bc[j] = 0;
        ck[j] = 0;
        if (ok[j]) ck[j] = dchain(key, (unsigned long long)(uint32_t)v[j]);
      }
#pragma unroll 1
      for (int j = 0; j < 4; ++j)
        if (ok[j]) {
          const int64_t bc = d_binomial_ool(ck[j], Bn, T);
          Bc[j] = (unsigned long long)bc;
          ok[j] = bc > 0;
        }
      if (__any_sync(FULL, ok[0] || ok[1] || ok[2] || ok[3])) {  // membership in the other backward lists
        const int drv = S.drv;
        for (int b = 0; b < nb; ++b) {
          if (b == drv) continue;
          const LR Lb = view_of(A.vdesc, A.drec, A.dlist, W.f[Lp.bpos[b]], Lp.bview[b]);
          const int32_t *bm = S.pm[b];
          walg += 4ull * (Lb.ml + Lb.xl);  // probed (binary search: an upper bound of the bytes it needs)
#pragma unroll 1
          for (int j = 0; j < 4; ++j)
            if (ok[j]) ok[j] = probe(A, W.f[Lp.bpos[b]], bm, Lb.ml, v[j]) || (Lb.xl && has(Lb.x, Lb.xl, v[j]));
        }
      }
      // whole chunks while their survivors fit the 32-entry buffer (chunk 0 always does); the rest is redone
      unsigned msk[4];
#pragma unroll
      for (int j = 0; j < 4; ++j) msk[j] = __ballot_sync(FULL, ok[j]);
      int taken = 0, tot = 0;
      int basej[4] = {0, 0, 0, 0};
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const int c = __popc(msk[j]);
        if (taken == j && (j == 0 || tot + c <= 32)) {
          basej[j] = tot;
          tot += c;
          taken = j + 1;
        }
      }
      __syncwarp();
#pragma unroll
      for (int j = 0; j < 4; ++j)
        if (j < taken && ok[j]) {
          const int r = basej[j] + __popc(msk[j] & ((1u << lane) - 1u));
          S.sv[r] = v[j];
          S.sB[r] = Bc[j];
          S.skey[r] = ck[j];
        }
      {
        unsigned long long sb = 0;
#pragma unroll
        for (int j = 0; j < 4; ++j)
          if (j < taken && ok[j]) sb += Bc[j];
        rec_shared(A, P, W.f, level, sb, lane);
      }
      if (lane == 0) {
        S.ns = tot;
        S.si = 0;
        S.pos = (int32_t)(pos + 32 * taken);
      }
      __syncwarp();
    }
  }
}

// ---- touched set, scores ----------------------------------------------------------------------------------

__global__ void k_clear_rows(const int32_t *tids, const SelState *st, unsigned long long *lev, int levels) {
  const unsigned long long n = st->n_touched;
  for (unsigned long long i = blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x; i < n;
       i += (unsigned long long)gridDim.x * blockDim.x)
    for (int l = 0; l < levels; ++l) lev[(size_t)tids[i] * levels + l] = 0;
}

__global__ void k_deg_bits(const VDesc *vdesc, int32_t n, uint32_t *touched) {
  const int64_t W = ((int64_t)n + 31) / 32;
  for (int64_t w = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; w < W; w += (int64_t)gridDim.x * blockDim.x) {
    uint32_t bits = 0;
    for (int b = 0; b < 32; ++b) {
      const int64_t v = w * 32 + b;
      if (v < n && vdesc[v].len > 0) bits |= 1u << b;
    }
    touched[w] = bits;
  }
}

__global__ void k_wcount(const uint32_t *touched, int64_t W, uint32_t *wcnt) {
  for (int64_t w = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; w <= W; w += (int64_t)gridDim.x * blockDim.x)
    wcnt[w] = w < W ? __popc(touched[w]) : 0u;
}

__global__ void k_wwrite(const uint32_t *touched, int64_t W, const uint32_t *woff, int32_t *tids, SelState *st) {
  for (int64_t w = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; w < W; w += (int64_t)gridDim.x * blockDim.x) {
    uint32_t bits = touched[w];
    uint32_t o = woff[w];
    while (bits) {
      const int b = __ffs(bits) - 1;
      tids[o++] = (int32_t)(w * 32 + b);
      bits &= bits - 1;
    }
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    st->n_touched = woff[W];
    st->above = 0;
    st->prefix = 0;
    st->mask = 0;
    st->found = 1;
    st->sel_bytes = 0;
  }
}

struct ScoreArgs {
  int32_t nq;
  int32_t policy;
  const unsigned long long *lev[GCSM_MAX_QUERIES];
  int32_t levels[GCSM_MAX_QUERIES];
  double N1[GCSM_MAX_QUERIES], M[GCSM_MAX_QUERIES];
  double powD[GCSM_MAX_QUERIES][8];
};

// eq. (3) averaged over M (estimator.cpp estimate_value), summed over the queries in registration order
__global__ void k_score(const ScoreArgs S, const int32_t *tids, const SelState *st, const VDesc *vdesc,
                        unsigned long long *bits, unsigned long long *bytes) {
  const unsigned long long n = st->n_touched;
  for (unsigned long long i = blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x; i < n;
       i += (unsigned long long)gridDim.x * blockDim.x) {
    const int32_t v = tids[i];
    const uint32_t len = vdesc[v].len;
    double s = 0.0;
    if (S.policy == 2) {
      s = (double)len;
    } else {
      for (int q = 0; q < S.nq; ++q) {
        const int L = S.levels[q];
        const unsigned long long *lv = S.lev[q] + (size_t)v * L;
        double e = 0.0;
        for (int l = 0; l < L; ++l) e = DA(e, DM(DM(S.N1[q], S.powD[q][l]), (double)lv[l]));
        e = DV(e, S.M[q]);
        s = DA(s, e);
      }
    }
    if (vdesc[v].upd != 0) s = 0.0;  // x ∈ U: S(x) is already in HBM with the batch (R32), it takes no budget
    bits[i] = (unsigned long long)__double_as_longlong(s);
    bytes[i] = (unsigned long long)((len + 3u) & ~3u) * 4ull;
  }
}

// ---- the ranking cut (R23) without a sort --------------------------------------------------------------------

__device__ __forceinline__ int cut_shift(int level) { return level < 5 ? 52 - 12 * level : 0; }
__device__ __forceinline__ unsigned long long cut_wmask(int level) { return level < 5 ? 4095ull : 15ull; }

__global__ void __launch_bounds__(256) k_hist(const unsigned long long *bits, const unsigned long long *bytes,
                                              const SelState *st, unsigned long long *hist, int level) {
  __shared__ unsigned long long h[4096];
  for (int i = threadIdx.x; i < 4096; i += blockDim.x) h[i] = 0;
  __syncthreads();
  const unsigned long long n = st->n_touched, mask = st->mask, prefix = st->prefix;
  const int sh = cut_shift(level);
  const unsigned long long wm = cut_wmask(level);
  if (st->found)
    for (unsigned long long i = blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x; i < n;
         i += (unsigned long long)gridDim.x * blockDim.x) {
      const unsigned long long b = bits[i];
      if ((long long)b > 0 && (b & mask) == prefix && bytes[i]) atomicAdd(&h[(b >> sh) & wm], bytes[i]);
    }
  __syncthreads();
  for (int i = threadIdx.x; i < 4096; i += blockDim.x)
    if (h[i]) atomicAdd(hist + (size_t)level * 4096 + i, h[i]);
}

// One block of 1024 threads: bins in descending order, 4 per thread; the first bin where the cumulative bytes
// pass the budget is the cut bucket of this level.
__global__ void __launch_bounds__(1024) k_cut(const unsigned long long *hist, SelState *st, uint64_t budget, int level) {
  __shared__ unsigned long long wsum[32];
  __shared__ int win;
  if (!st->found) return;
  if (threadIdx.x == 0) win = 1 << 30;
  const unsigned long long *h = hist + (size_t)level * 4096;
  const int nbins = level < 5 ? 4096 : 16;
  unsigned long long v[4], tot = 0;
  for (int j = 0; j < 4; ++j) {
    const int d = 4 * threadIdx.x + j;  // descending position
    v[j] = d < nbins ? h[nbins - 1 - d] : 0ull;
    tot += v[j];
  }
  // exclusive block scan of the per-thread totals (warp shuffles, then the 32 warp totals)
  const int lane = threadIdx.x & 31, wi = threadIdx.x >> 5;
  unsigned long long x = tot;
  for (int o = 1; o < 32; o <<= 1) {
    const unsigned long long y = __shfl_up_sync(FULL, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) wsum[wi] = x;
  __syncthreads();
  if (wi == 0) {
    unsigned long long t = wsum[lane];
    for (int o = 1; o < 32; o <<= 1) {
      const unsigned long long y = __shfl_up_sync(FULL, t, o);
      if (lane >= o) t += y;
    }
    wsum[lane] = t;
  }
  __syncthreads();
  const unsigned long long before = x - tot + (wi ? wsum[wi - 1] : 0ull);
  __syncthreads();
  const unsigned long long above = st->above;
  unsigned long long cum = above + before;
  int mine = -1;
  unsigned long long mine_cum = 0;
  for (int j = 0; j < 4; ++j) {
    if (cum + v[j] > budget) {
      mine = 4 * threadIdx.x + j;
      mine_cum = cum;
      break;
    }
    cum += v[j];
  }
  if (mine >= 0) atomicMin(&win, mine);
  __syncthreads();
  if (mine >= 0 && mine == win) {
    const int bin = nbins - 1 - mine;
    const int sh = cut_shift(level);
    st->prefix |= (unsigned long long)bin << sh;
    st->mask |= cut_wmask(level) << sh;
    st->above = mine_cum;
  }
  if (threadIdx.x == 0 && win == (1 << 30)) st->found = 0;  // everything fits (level 0)
}

__global__ void k_ties(const unsigned long long *bits, const unsigned long long *bytes, const SelState *st, int64_t cap,
                       unsigned long long *out) {
  const unsigned long long n = st->n_touched;
  const bool found = st->found != 0;
  const unsigned long long prefix = st->prefix;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < cap; i += (int64_t)gridDim.x * blockDim.x)
    out[i] = ((unsigned long long)i < n && found && bits[i] == prefix) ? bytes[i] : 0ull;
}

// selection flag; scan[i] (tie prefix in, selected bytes out)
__global__ void k_select(const unsigned long long *bits, const unsigned long long *bytes, SelState *st, int64_t cap,
                         uint64_t budget, unsigned long long *scan, uint8_t *flag) {
  const unsigned long long n = st->n_touched;
  const bool found = st->found != 0;
  const unsigned long long prefix = st->prefix, above = st->above;
  unsigned long long used = 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < cap; i += (int64_t)gridDim.x * blockDim.x) {
    bool sel = false;
    if ((unsigned long long)i < n) {
      const unsigned long long b = bits[i];
      sel = (long long)b > 0 && (!found || b > prefix || (b == prefix && above + scan[i] <= budget));
    }
    flag[i] = sel;
    const unsigned long long sb = sel ? bytes[i] : 0ull;
    scan[i] = sb;
    used += sb;
  }
  for (int o = 16; o; o >>= 1) used += __shfl_xor_sync(FULL, used, o);
  if ((threadIdx.x & 31) == 0 && used) atomicAdd(&st->sel_bytes, used);
}

// warp per 32 touched entries: copy each selected list (16-byte granules) from where its descriptor points
__global__ void __launch_bounds__(256) k_copy(const int32_t *tids, const SelState *st, const uint8_t *flag,
                                              const unsigned long long *off, const unsigned long long *bytes,
                                              const VDesc *vdesc, char *cache) {
  const unsigned long long n = st->n_touched;
  const int lane = threadIdx.x & 31;
  const unsigned long long nw = (unsigned long long)gridDim.x * (blockDim.x >> 5);
  for (unsigned long long base = ((unsigned long long)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5)) * 32;
       base < n; base += nw * 32) {
    const unsigned long long i = base + lane;
    const bool sel = i < n && flag[i];
    unsigned mask = __ballot_sync(FULL, sel);
    while (mask) {
      const int j = __ffs(mask) - 1;
      mask &= mask - 1;
      const unsigned long long e = base + j;
      const int32_t v = tids[e];
      const uint4 *src = reinterpret_cast<const uint4 *>(vdesc[v].ptr);
      uint4 *dst = reinterpret_cast<uint4 *>(cache + off[e]);
      const unsigned long long g = bytes[e] / 16;
      unsigned long long t = lane;
      for (; t + 96 < g; t += 128) {  // 4 x 16 B loads in flight per lane
        const uint4 a = src[t], b = src[t + 32], c = src[t + 64], d = src[t + 96];
        dst[t] = a;
        dst[t + 32] = b;
        dst[t + 64] = c;
        dst[t + 96] = d;
      }
      for (; t < g; t += 32) dst[t] = src[t];
    }
  }
}

__global__ void k_reset_prev(const int32_t *prev, const SelState *st, VDesc *vdesc, const unsigned long long *hptr) {
  const unsigned long long n = st->prev_sel;
  for (unsigned long long i = blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x; i < n;
       i += (unsigned long long)gridDim.x * blockDim.x) {
    const int32_t v = prev[i];
    vdesc[v].ptr = reinterpret_cast<const int32_t *>(hptr[v]);
  }
}

__global__ void k_set_new(const int32_t *tids, const SelState *st, const uint8_t *flag, const unsigned long long *off,
                          VDesc *vdesc, char *cache) {
  const unsigned long long n = st->n_touched;
  for (unsigned long long i = blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x; i < n;
       i += (unsigned long long)gridDim.x * blockDim.x)
    if (flag[i]) vdesc[tids[i]].ptr = reinterpret_cast<const int32_t *>(cache + off[i]);
}

__global__ void k_sel_stats(SelState *st, unsigned long long *cnt, int has_cache) {
  if (!has_cache) {
    st->prev_sel = 0;
    st->sel_bytes = 0;
  }
  cnt[0] = st->prev_sel;
  cnt[1] = st->sel_bytes;
  cnt[2] = (unsigned long long)st->err;
}

__global__ void k_zero_touched_count(SelState *st) { st->n_touched = 0; }

__global__ void k_patch_host(VDesc *vdesc, unsigned long long *hptr, const int64_t *idx, const VDesc *val, int64_t n) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t v = idx[i];
    vdesc[v] = val[i];
    hptr[v] = (unsigned long long)val[i].ptr;
  }
}

__global__ void k_est_gather(const int32_t *tids, int64_t n, const unsigned long long *lev, int levels,
                             unsigned long long *out) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    for (int l = 0; l < 8; ++l) out[i * 8 + l] = l < levels ? lev[(size_t)tids[i] * levels + l] : 0ull;
}

int gs_grid(int64_t n, int per = 256) { return (int)std::max<int64_t>(1, std::min<int64_t>((n + per - 1) / per, 148 * 8)); }

// ---- device-wide scans and the flagged select of the ranking (hand-written; three passes: 2048-element block
// scans, one block scanning the block totals, the carries added back). The element count is the host bound n,
// or the device-resident count *nd when given (the batch's touched set), so only live elements are scanned.
constexpr int kScanT = 256, kScanIt = 8, kScanBlk = kScanT * kScanIt;

__device__ __forceinline__ int64_t live_n(const unsigned long long *nd, int64_t n) {
  return nd ? (int64_t)min((unsigned long long)n, *nd) : n;
}

template <typename T>
__global__ void __launch_bounds__(kScanT) k_scan_blocks(const T *in, T *out, const unsigned long long *nd, int64_t nmax,
                                                        T *bsum, int inclusive) {
  __shared__ T ws[kScanT / 32];
  const int64_t n = live_n(nd, nmax);
  const int64_t base = (int64_t)blockIdx.x * kScanBlk + (int64_t)threadIdx.x * kScanIt;
  T v[kScanIt], run = 0;
#pragma unroll
  for (int i = 0; i < kScanIt; ++i) {
    const T x = base + i < n ? in[base + i] : (T)0;
    v[i] = inclusive ? run + x : run;
    run += x;
  }
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  T xs = run;  // inclusive scan of the per-thread totals in the warp
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const T y = __shfl_up_sync(FULL, xs, o);
    if (lane >= o) xs += y;
  }
  if (lane == 31) ws[w] = xs;
  __syncthreads();
  if (w == 0) {
    T t = lane < kScanT / 32 ? ws[lane] : (T)0;
#pragma unroll
    for (int o = 1; o < kScanT / 32; o <<= 1) {
      const T y = __shfl_up_sync(FULL, t, o);
      if (lane >= o) t += y;
    }
    if (lane < kScanT / 32) ws[lane] = t;
  }
  __syncthreads();
  const T excl = xs - run + (w ? ws[w - 1] : (T)0);
#pragma unroll
  for (int i = 0; i < kScanIt; ++i)
    if (base + i < n) out[base + i] = v[i] + excl;
  if (threadIdx.x == kScanT - 1) bsum[blockIdx.x] = excl + run;  // 0 for blocks past the live count
}

template <typename T>
__global__ void __launch_bounds__(1024) k_scan_totals(T *bsum, int64_t nb) {  // exclusive, in place
  __shared__ T ws[32];
  __shared__ T carry;
  if (threadIdx.x == 0) carry = 0;
  __syncthreads();
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  for (int64_t s0 = 0; s0 < nb; s0 += 1024) {
    const int64_t i = s0 + threadIdx.x;
    const T v = i < nb ? bsum[i] : (T)0;
    T x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const T y = __shfl_up_sync(FULL, x, o);
      if (lane >= o) x += y;
    }
    if (lane == 31) ws[w] = x;
    __syncthreads();
    if (w == 0) {
      T t = ws[lane];
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const T y = __shfl_up_sync(FULL, t, o);
        if (lane >= o) t += y;
      }
      ws[lane] = t;
    }
    __syncthreads();
    const T incl = x + (w ? ws[w - 1] : (T)0);
    if (i < nb) bsum[i] = carry + incl - v;
    __syncthreads();
    if (threadIdx.x == 1023) carry += incl;
    __syncthreads();
  }
}

template <typename T>
__global__ void k_scan_carry(T *out, const unsigned long long *nd, int64_t nmax, const T *bsum) {
  const int64_t n = live_n(nd, nmax);
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    out[i] += bsum[i / kScanBlk];
}

template <typename T>
cudaError_t scan(const T *in, T *out, const unsigned long long *nd, int64_t nmax, bool inclusive, void *tmp,
                 cudaStream_t s, uint64_t &L) {
  if (nmax <= 0) return cudaSuccess;
  const int64_t nb = (nmax + kScanBlk - 1) / kScanBlk;
  T *bsum = reinterpret_cast<T *>(tmp);
  k_scan_blocks<T><<<(unsigned)nb, kScanT, 0, s>>>(in, out, nd, nmax, bsum, inclusive ? 1 : 0);
  k_scan_totals<T><<<1, 1024, 0, s>>>(bsum, nb);
  k_scan_carry<T><<<gs_grid(nmax), 256, 0, s>>>(out, nd, nmax, bsum);
  L += 3;
  return cudaGetLastError();
}

// out[pos(i)] = in[i] for the flagged i < n (order kept), *count = their number; pos = exclusive scan of the flags
__global__ void k_flags_u32(const uint8_t *flag, uint32_t *f32, const unsigned long long *nd, int64_t nmax) {
  const int64_t n = live_n(nd, nmax);
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    f32[i] = flag[i] ? 1u : 0u;
}

__global__ void k_select_scatter(const int32_t *in, const uint8_t *flag, const uint32_t *pos,
                                 const unsigned long long *nd, int64_t nmax, int32_t *out, unsigned long long *count) {
  const int64_t n = live_n(nd, nmax);
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    if (flag[i]) out[pos[i]] = in[i];
    if (i == n - 1) *count = (unsigned long long)pos[i] + (flag[i] ? 1ull : 0ull);
  }
  if (blockIdx.x == 0 && threadIdx.x == 0 && n == 0) *count = 0;
}

}  // namespace

size_t cache_step_tmp_bytes(int32_t n) {
  // the scans' block totals (u64), then the select's u32 flags and positions
  const size_t nb = ((size_t)n + 2 + kScanBlk - 1) / kScanBlk + 1;
  return 8 * nb + 8 * ((size_t)n + 2) + 256;
}

cudaError_t launch_patch_vdesc_host(VDesc *vdesc, unsigned long long *hptr, const int64_t *idx, const VDesc *val,
                                    int64_t n, cudaStream_t s) {
  if (n <= 0) return cudaSuccess;
  k_patch_host<<<gs_grid(n), 256, 0, s>>>(vdesc, hptr, idx, val, n);
  return cudaGetLastError();
}

cudaError_t launch_estimates_gather(const int32_t *tids, int64_t n, const unsigned long long *levcnt, int levels,
                                    unsigned long long *lev_out, cudaStream_t s) {
  if (n <= 0) return cudaSuccess;
  k_est_gather<<<gs_grid(n), 256, 0, s>>>(tids, n, levcnt, levels, lev_out);
  return cudaGetLastError();
}

cudaError_t launch_cache_step(const CacheStep &c, cudaStream_t s, uint64_t *launches) {
  const int64_t n = c.n, W = (n + 31) / 32;
  const int G = 148 * 4;
  uint64_t L = 0;
  cudaError_t e;
#define LK(...)                              \
  do {                                       \
    __VA_ARGS__;                             \
    if ((e = cudaGetLastError()) != cudaSuccess) return e; \
    ++L;                                     \
  } while (0)
  if (c.reset_first) {
    LK(k_reset_prev<<<G, 256, 0, s>>>(c.prev_sel, c.st, c.vdesc, c.hptr));
    if ((e = cudaMemsetAsync(&c.st->prev_sel, 0, sizeof(unsigned long long), s)) != cudaSuccess) return e;
  }
  // last batch's estimator sums are cleared (rows of its touched set)
  for (int q = 0; q < c.nq; ++q)
    if (c.q[q].levcnt && c.q[q].k > 2) LK(k_clear_rows<<<G, 256, 0, s>>>(c.tids, c.st, c.q[q].levcnt, c.q[q].k - 2));
  if (c.policy == 0) {
    LK(k_zero_touched_count<<<1, 1, 0, s>>>(c.st));
    LK(k_reset_prev<<<G, 256, 0, s>>>(c.prev_sel, c.st, c.vdesc, c.hptr));
    LK(k_sel_stats<<<1, 1, 0, s>>>(c.st, c.cnt_cached, 0));
    *launches += L;
    return cudaSuccess;
  }
  if ((e = cudaMemsetAsync(c.touched, 0, sizeof(uint32_t) * (size_t)W, s)) != cudaSuccess) return e;
  if (c.policy == 2) {
    LK(k_deg_bits<<<gs_grid(W), 256, 0, s>>>(c.vdesc, c.n, c.touched));
  } else {
    if ((e = cudaMemsetAsync(c.cursor, 0, sizeof(unsigned long long) * 3 * c.nq, s)) != cudaSuccess) return e;
    for (int q = 0; q < c.nq; ++q) {
      const EstQuery &Q = c.q[q];
      if (Q.k <= 2 || Q.n_units <= 0) continue;
      WalkArgs A;
      A.plans = Q.plans;
      A.units = Q.units;
      A.n_units = Q.n_units;
      A.items = Q.items;
      A.n_items = Q.n_items;
      A.f2 = c.f2;
      A.f2_cap = Q.f2_cap;
      A.f2_count = c.cursor + 3 * q + 2;
      A.cursor2 = c.cursor + 3 * q + 1;
      A.levcnt = Q.levcnt;
      A.levels = Q.k - 2;
      A.vdesc = c.vdesc;
      A.drec = c.drec;
      A.dlist = c.dlist;
      A.lab = c.lab;
      A.touched = c.touched;
      A.cursor = c.cursor + 3 * q;
      A.T.pD = c.pD;
      A.T.r0tab = c.r0tab;
      A.T.r0n = c.r0n;
      A.T.sfc = c.sfc_dev;
      A.T.err = &c.st->err;
      A.stage = c.stage;
      A.stage_min = c.stage_min;
      A.stage_cnt = c.stage_cnt;
      A.alg_cnt = c.alg_cnt[q];
      A.walk_stage = c.walk_stage;
      A.lane_leaf = c.walk_lane;
      A.sidx = c.sidx;
      A.soff = c.soff;
      for (int r = 0; r < 2; ++r) {
        A.dev_lo[r] = c.dev_lo[r];
        A.dev_hi[r] = c.dev_hi[r];
      }
      const int ga = (int)std::max<int64_t>(1, std::min<int64_t>((Q.n_items + kEW - 1) / kEW, 148 * 8));
      if (c.ev_walk && q < GCSM_MAX_QUERIES) cudaEventRecord(c.ev_walk[2 * q], s);
      LK(k_walks_l1<<<ga, kEW * 32, 0, s>>>(A));
      if (Q.k >= 5) LK(k_walks<<<148 * GCSM_WALK_MINBLOCKS, kEW * 32, 0, s>>>(A));
      if (c.ev_walk && q < GCSM_MAX_QUERIES) cudaEventRecord(c.ev_walk[2 * q + 1], s);
    }
  }
  // touched set in id order
  uint32_t *wcnt = c.wcnt;
  uint32_t *woff = c.woff;
  LK(k_wcount<<<gs_grid(W + 1), 256, 0, s>>>(c.touched, W, wcnt));
  if ((e = scan<uint32_t>(wcnt, woff, nullptr, W + 1, false, c.cub_tmp, s, L)) != cudaSuccess) return e;
  LK(k_wwrite<<<gs_grid(W), 256, 0, s>>>(c.touched, W, woff, c.tids, c.st));
  ScoreArgs S{};
  S.nq = c.nq;
  S.policy = c.policy;
  for (int q = 0; q < c.nq; ++q) {
    S.lev[q] = c.q[q].levcnt;
    S.levels[q] = c.q[q].k > 2 ? c.q[q].k - 2 : 0;
    S.N1[q] = (double)c.q[q].N1;
    S.M[q] = (double)c.q[q].M;
    for (int l = 0; l < 8; ++l) S.powD[q][l] = c.q[q].powD[l];
    if (!c.q[q].levcnt || c.q[q].n_units <= 0) S.levels[q] = 0, S.M[q] = 1.0;
  }
  LK(k_score<<<G, 256, 0, s>>>(S, c.tids, c.st, c.vdesc, c.bits, c.bytes));
  if ((e = cudaMemsetAsync(c.hist, 0, sizeof(unsigned long long) * 6 * 4096, s)) != cudaSuccess) return e;
  for (int lv = 0; lv < 6; ++lv) {
    LK(k_hist<<<G, 256, 0, s>>>(c.bits, c.bytes, c.st, c.hist, lv));
    LK(k_cut<<<1, 1024, 0, s>>>(c.hist, c.st, c.budget, lv));
  }
  LK(k_ties<<<G, 256, 0, s>>>(c.bits, c.bytes, c.st, n, c.off));
  if ((e = scan<unsigned long long>(c.off, c.scan, &c.st->n_touched, n, true, c.cub_tmp, s, L)) != cudaSuccess)
    return e;
  LK(k_select<<<G, 256, 0, s>>>(c.bits, c.bytes, c.st, n, c.budget, c.scan, c.flag));
  if ((e = scan<unsigned long long>(c.scan, c.off, &c.st->n_touched, n, false, c.cub_tmp, s, L)) != cudaSuccess)
    return e;
  LK(k_copy<<<G, 256, 0, s>>>(c.tids, c.st, c.flag, c.off, c.bytes, c.vdesc, c.cache));
  LK(k_reset_prev<<<G, 256, 0, s>>>(c.prev_sel, c.st, c.vdesc, c.hptr));
  LK(k_set_new<<<G, 256, 0, s>>>(c.tids, c.st, c.flag, c.off, c.vdesc, c.cache));
  {  // the selection, compacted in id order (the next batch's previous selection)
    const size_t nb = ((size_t)n + kScanBlk - 1) / kScanBlk + 1;
    uint32_t *f32 = reinterpret_cast<uint32_t *>(reinterpret_cast<char *>(c.cub_tmp) + 8 * nb);
    uint32_t *pos = f32 + (n + 1);  // two u32 arrays of n + 1 in the 8 (n + 2) bytes
    LK(k_flags_u32<<<gs_grid(n), 256, 0, s>>>(c.flag, f32, &c.st->n_touched, n));
    if ((e = scan<uint32_t>(f32, pos, &c.st->n_touched, n, false, c.cub_tmp, s, L)) != cudaSuccess) return e;
    LK(k_select_scatter<<<gs_grid(n), 256, 0, s>>>(c.tids, c.flag, pos, &c.st->n_touched, n, c.prev_sel,
                                                  &c.st->prev_sel));
  }
  LK(k_sel_stats<<<1, 1, 0, s>>>(c.st, c.cnt_cached, 1));
#undef LK
  *launches += L;
  return cudaSuccess;
}

}  // namespace gcsm
