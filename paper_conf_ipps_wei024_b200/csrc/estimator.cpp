// estimator.cpp — random-walk access-frequency estimation (step ②, §IV).
//
// a walk picks a level-1 node (updated edge) w.p. 1/|ΔE|, then a child
// uniformly from the node's candidate set V and continues w.p. |V|/D, i.e.
// every child w.p. 1/D. Eq. (3): C~_v = Σ_i |ΔE| D^{i-1} c_{v,i},
// averaged over M walks. §IV-B: the M walks are merged into one
// execution of the nested loops — a level-1 node is visited B_1 ~ Bin(M,
// 1/|ΔE|) times, a child of a node visited B times B' ~ Bin(B, 1/D) times,
// nodes with B = 0 are skipped, and the per-vertex sums are kept in O(|V|).
// Readings: R15 (|ΔE| = N1 = #units), R16 (forest of all terms), R17 (a node
// at level l reads the lists of the next position's backward neighbours),
// R18 (V after label/injectivity filters), R19 (D = max list length over
// G_t ∪ G_{t+1}), R20 (independent binomials), R21 (M of P:339),
// R22 (counter-based keys: identical results for any thread count).
//
// Output: for every vertex read at least once, Σ B per tree level l = 1..k-2.
// Implementation notes (exact reorderings, same distribution and same draws):
//  * in the inversion branch (B/D < 10) the children with B' > 0 are found by
//    skip sampling (geometric gaps over segments of the driver, then B' drawn
//    conditioned on >= 1): the same law as one independent binomial per child,
//    with work proportional to the children drawn, not to the driver (skip_gap).

#include <algorithm>
#include <cmath>
#include <cstring>
#include <memory>

#include "estimator.h"

namespace gcsm {

uint64_t rng_mix(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}

uint64_t rng_chain(uint64_t h, uint64_t x) { return rng_mix(h + 0x9E3779B97F4A7C15ULL * (x + 1)); }

namespace {

struct Uniforms {
  uint64_t key;
  uint64_t j = 0;
  double next() {
    ++j;
    return (double)(rng_mix(key + 0xD1B54A32D192ED03ULL * j) >> 11) * (1.0 / 9007199254740992.0);
  }
};

double stirling_fc(int64_t k) {
  if (k < 10) {
    const double kk = (double)k;
    return std::lgamma(kk + 1.0) - ((kk + 0.5) * std::log(kk + 1.0) - (kk + 1.0) + 0.5 * std::log(2.0 * M_PI));
  }
  const double r = 1.0 / (double)(k + 1), r2 = r * r;
  return (1.0 / 12.0 - (1.0 / 360.0 - (1.0 / 1260.0) * r2) * r2) * r;
}

// Inversion (Kachitvichyanukul & Schmeiser BINV) for n p < 10.
int64_t binv(Uniforms &U, int64_t n, double p) {
  const double q = 1.0 - p;
  const double s = p / q, a = (double)(n + 1) * s;
  const double r0 = std::pow(q, (double)n);
  for (;;) {
    double r = r0, u = U.next();
    int64_t x = 0;
    while (u > r) {
      u -= r;
      x += 1;
      if (x > n) break;
      r *= (a / (double)x - s);
    }
    if (x <= n) return x;
  }
}

// Transformed rejection with decomposition (Hörmann 1993, BTRD) for n p >= 10.
int64_t btrd(Uniforms &U, int64_t n, double p) {
  const double q = 1.0 - p;
  const double m = std::floor((double)(n + 1) * p);
  const double r = p / q, nr = (double)(n + 1) * r, npq = (double)n * p * q;
  const double spq = std::sqrt(npq);
  const double b = 1.15 + 2.53 * spq;
  const double a = -0.0873 + 0.0248 * b + 0.01 * p;
  const double c = (double)n * p + 0.5;
  const double alpha = (2.83 + 5.1 / b) * spq;
  const double vr = 0.92 - 4.2 / b;
  const double urvr = 0.86 * vr;
  const int64_t mi = (int64_t)m;
  for (;;) {
    double v = U.next(), u;
    if (v <= urvr) {
      u = v / vr - 0.43;
      return (int64_t)std::floor((2.0 * a / (0.5 - std::fabs(u)) + b) * u + c);
    }
    if (v >= vr) {
      u = U.next() - 0.5;
    } else {
      u = v / vr - 0.93;
      u = (u < 0 ? -0.5 : 0.5) - u;
      v = U.next() * vr;
    }
    const double us = 0.5 - std::fabs(u);
    const double kd = std::floor((2.0 * a / us + b) * u + c);
    if (kd < 0.0 || kd > (double)n) continue;
    const int64_t ki = (int64_t)kd;
    v = v * alpha / (a / (us * us) + b);
    const int64_t km = ki > mi ? ki - mi : mi - ki;
    if (km <= 15) {
      double f = 1.0;
      if (mi < ki) {
        for (int64_t i = mi + 1; i <= ki; ++i) f *= (nr / (double)i - r);
      } else if (mi > ki) {
        for (int64_t i = ki + 1; i <= mi; ++i) v *= (nr / (double)i - r);
      }
      if (v <= f) return ki;
      continue;
    }
    v = std::log(v);
    const double kmd = (double)km;
    const double rho = (kmd / npq) * (((kmd / 3.0 + 0.625) * kmd + 1.0 / 6.0) / npq + 0.5);
    const double t = -kmd * kmd / (2.0 * npq);
    if (v < t - rho) return ki;
    if (v > t + rho) continue;
    const double nm = (double)(n - mi + 1);
    const double h = (m + 0.5) * std::log((m + 1.0) / (r * nm)) + stirling_fc(mi) + stirling_fc(n - mi);
    const double nk = (double)(n - ki + 1);
    if (v <= h + (double)(n + 1) * std::log(nm / nk) + (kd + 0.5) * std::log(nk * r / (kd + 1.0)) -
                 stirling_fc(ki) - stirling_fc(n - ki))
      return ki;
  }
}

}  // namespace

int64_t binomial(uint64_t key, int64_t n, double p) {
  if (n <= 0 || p <= 0.0) return 0;
  if (p >= 1.0) return n;
  Uniforms U{key};
  if (p > 0.5) {
    const double pp = 1.0 - p;
    return n - ((double)n * pp < 10.0 ? binv(U, n, pp) : btrd(U, n, pp));
  }
  return (double)n * p < 10.0 ? binv(U, n, p) : btrd(U, n, p);
}

double stirling_small(int k) { return stirling_fc(k); }

// ---- skip sampling of a node's children in BINV's domain -------------------------------------
// Every child of a node with multiplicity B draws B' ~ Bin(B, p), p = 1/D, independently (R20); in BINV's domain
// B' > 0 has probability q = 1 - r0, r0 = (1-p)^B, which is small at levels >= 2 (C4: ~2.5 %). Instead of one
// coin per driver element, the driver is cut into segments of kSkipSeg elements and each segment's selected
// elements are found by geometric gaps G with P(G >= g) = r0^g (iid Bernoulli(q) per element), drawn from the
// segment's own counter stream; a selected element that is a child then draws B' from Bin(B, p) conditioned on
// B' >= 1 (its own stream, keyed by the child as before). The law of the children's draws is exactly the
// independent binomials' — only the random numbers differ. The device walker computes the same doubles in the
// same order (round-to-nearest, no contraction), so both draw the same children.
int64_t binom_pos(uint64_t ck, int64_t n, double p, double r0) {
  Uniforms U{ck};
  const double q = 1.0 - p, s = p / q, a = (double)(n + 1) * s;
  for (;;) {
    double u = r0 + (1.0 - r0) * U.next();  // uniform on (r0, 1]: the inversion never stops at 0
    double r = r0;
    int64_t x = 0;
    while (u > r) {
      u -= r;
      x += 1;
      if (x > n) break;
      r *= (a / (double)x - s);
    }
    if (x > n) continue;
    return x < 1 ? 1 : x;
  }
}

void skip_table(double r0, double *pw) {
  pw[0] = r0;
  for (int i = 1; i < kSkipLog + 1; ++i) pw[i] = pw[i - 1] * pw[i - 1];
}

uint32_t skip_gap(const double *pw, double u) {  // the largest g < 2 kSkipSeg with r0^g >= u
  double cur = 1.0;
  uint32_t g = 0;
  for (int i = kSkipLog; i >= 0; --i) {
    const double c = cur * pw[i];
    if (c >= u) {
      cur = c;
      g += 1u << i;
    }
  }
  return g;
}

uint64_t skip_uniform_bits(uint64_t segkey, uint64_t j) { return rng_mix(segkey + 0xD1B54A32D192ED03ULL * j) >> 11; }

uint64_t walk_budget(uint64_t N1, uint64_t D, int k) {
  // M = floor(N1 * D^(k-2) / 32^k), clamped to [1, 2^62] (R21), exact integer arithmetic.
  if (N1 == 0) return 1;
  const unsigned __int128 cap = (unsigned __int128)1 << 62;
  unsigned __int128 num = N1;
  for (int i = 0; i < k - 2; ++i) {
    num *= D;
    if (num > cap * ((unsigned __int128)1 << 40)) return (uint64_t)cap;
  }
  unsigned __int128 den = 1;
  for (int i = 0; i < k; ++i) den *= 32;
  unsigned __int128 M = num / den;
  if (M < 1) M = 1;
  if (M > cap) M = cap;
  return (uint64_t)M;
}

namespace {

constexpr int kPartLog2 = 14;  // ids per reduction partition (16K x levels x 8 B stays in L2)

struct Walker {
  const EstimatorInput &in;
  EstimatorScratch &scr;
  const DevPlan *P = nullptr;
  int32_t f[GCSM_MAXK];
  std::vector<uint32_t> keep_[GCSM_MAXK];
  std::vector<EstRec> *out = nullptr;  // this thread's partition buffers
  Walker(const EstimatorInput &i, EstimatorScratch &s) : in(i), scr(s) {}

  bool member(const HList &L, int32_t v) const {
    return std::binary_search(L.a, L.a + L.na, v) || (L.nb && std::binary_search(L.b, L.b + L.nb, v));
  }

  void record(int32_t v, int level, uint64_t B) { out[(uint32_t)v >> kPartLog2].push_back({v, (uint32_t)level, B}); }

  // node at `level` (positions 0..level matched), multiplicity B, key
  void visit(int level, int64_t B, uint64_t key) {
    const int k = P->k;
    if (level >= k - 1) return;  // leaf: reads nothing
    const int p = level + 1;
    const LevelPlan &Lp = P->lv[p];
    HList L[7];
    for (int b = 0; b < Lp.nb; ++b) {
      L[b] = in.view(f[Lp.bpos[b]], Lp.bview[b]);
      record(f[Lp.bpos[b]], level, (uint64_t)B);
    }
    if (level == k - 2) return;  // children are leaves: they read nothing
    // candidates of position p, each child drawn B' ~ Bin(B, 1/D)
    int drv = 0;
    for (int b = 1; b < Lp.nb; ++b)
      if (L[b].na + L[b].nb < L[drv].na + L[drv].nb) drv = b;
    const double pD = 1.0 / (double)in.D;
    const bool fast = B > 0 && pD > 0.0 && pD <= 0.5 && (double)B * pD < 10.0;
    const double r0 = fast ? std::pow(1.0 - pD, (double)B) : 0.0;
    auto consider = [&](int32_t v) {
      for (int s = 0; s < p; ++s)
        if (f[s] == v) return;
      if (Lp.label >= 0 && (in.labels ? (int32_t)in.labels[v] : 0) != Lp.label) return;
      const uint64_t ck = rng_chain(key, (uint64_t)(uint32_t)v);
      for (int b = 0; b < Lp.nb; ++b)
        if (b != drv && !member(L[b], v)) return;
      const int64_t Bc = binomial(ck, B, pD);
      if (Bc <= 0) return;
      f[p] = v;
      visit(level + 1, Bc, ck);
    };
    if (fast) {  // skip sampling over segments of the driver (main then delta segment)
      auto consider_sel = [&](int32_t v) {
        for (int s = 0; s < p; ++s)
          if (f[s] == v) return;
        if (Lp.label >= 0 && (in.labels ? (int32_t)in.labels[v] : 0) != Lp.label) return;
        for (int b = 0; b < Lp.nb; ++b)
          if (b != drv && !member(L[b], v)) return;
        const uint64_t ck = rng_chain(key, (uint64_t)(uint32_t)v);
        const int64_t Bc = binom_pos(ck, B, pD, r0);
        f[p] = v;
        visit(level + 1, Bc, ck);
      };
      double pw[kSkipLog + 1];
      skip_table(r0, pw);
      const uint32_t na = L[drv].na, nd = na + L[drv].nb;
      for (uint32_t s0 = 0; s0 < nd; s0 += kSkipSeg) {
        const uint32_t s1 = std::min<uint32_t>(nd, s0 + kSkipSeg);
        const uint64_t segkey = rng_chain(key, kSkipTag + s0 / kSkipSeg);
        uint32_t pos = s0;
        for (uint64_t j = 1;; ++j) {
          const uint32_t g = skip_gap(pw, (double)skip_uniform_bits(segkey, j) * (1.0 / 9007199254740992.0));
          if (g >= s1 - pos) break;
          pos += g;
          consider_sel(pos < na ? L[drv].a[pos] : L[drv].b[pos - na]);
          if (++pos >= s1) break;
        }
      }
    } else {
      for (uint32_t i = 0; i < L[drv].na; ++i) consider(L[drv].a[i]);
      for (uint32_t i = 0; i < L[drv].nb; ++i) consider(L[drv].b[i]);
    }
  }
};

}  // namespace

void run_estimator(const EstimatorInput &in, EstimatorScratch &scr, EstimatorOutput &out) {
  out.ids.clear();
  out.levcnt.clear();
  const int k = in.plans[0].k;
  if (k <= 2 || in.n_units == 0) return;
  const int levels = k - 2;
  const int T = std::max(1, std::min(in.threads, pool_size()));
  const int parts = (int)(((int64_t)in.n + (1 << kPartLog2) - 1) >> kPartLog2);
  if (scr.n != in.n || scr.threads != T || scr.parts != parts) {
    scr.n = in.n;
    scr.threads = T;
    scr.parts = parts;
    scr.buf.assign((size_t)T * parts, {});
  }
  for (auto &b : scr.buf) b.clear();
  const uint64_t root = rng_mix(in.seed);
  const double p1 = 1.0 / (double)in.N1;
  std::vector<std::unique_ptr<Walker>> walkers(T);
  for (int t = 0; t < T; ++t) {
    walkers[t].reset(new Walker(in, scr));
    walkers[t]->out = &scr.buf[(size_t)t * parts];
  }
  parallel_dyn(T, in.n_units, 64, [&](int tid, int64_t ui) {
    const Unit &u = in.units[ui];
    const int term = u.plan >> 1, kind = u.plan & 1;
    const uint64_t key = rng_chain(rng_chain(rng_chain(rng_chain(rng_chain(root, in.batch_seq), (uint64_t)term),
                                                       (uint64_t)kind), (uint64_t)(uint32_t)u.a),
                                   (uint64_t)(uint32_t)u.b);
    const int64_t B = binomial(key, (int64_t)in.M, p1);
    if (B <= 0) return;
    Walker &w = *walkers[tid];
    w.P = &in.plans[u.plan];
    w.f[0] = u.a;
    w.f[1] = u.b;
    w.visit(1, B, key);
  });
  // reduce each vertex-range partition in a dense window (one thread per partition), ids in ascending order
  std::vector<std::vector<int32_t>> pid((size_t)parts);
  std::vector<std::vector<uint64_t>> plev((size_t)parts);
  parallel_dyn(T, parts, 1, [&](int, int64_t p) {
    size_t nrec = 0;
    for (int t = 0; t < T; ++t) nrec += scr.buf[(size_t)t * parts + p].size();
    if (!nrec) return;
    const int64_t base = p << kPartLog2;
    const int64_t span = std::min<int64_t>((int64_t)1 << kPartLog2, (int64_t)in.n - base);
    thread_local std::vector<uint64_t> win;
    thread_local std::vector<uint8_t> hit;
    win.assign((size_t)span * levels, 0);
    hit.assign((size_t)span, 0);
    for (int t = 0; t < T; ++t)
      for (const EstRec &r : scr.buf[(size_t)t * parts + p]) {
        const int64_t o = r.v - base;
        win[(size_t)o * levels + (r.level - 1)] += r.B;
        hit[o] = 1;
      }
    auto &ids = pid[p];
    auto &lev = plev[p];
    for (int64_t o = 0; o < span; ++o)
      if (hit[o]) {
        ids.push_back((int32_t)(base + o));
        for (int l = 0; l < 8; ++l) lev.push_back(l < levels ? win[(size_t)o * levels + l] : 0);
      }
  });
  std::vector<size_t> off((size_t)parts + 1, 0);
  for (int p = 0; p < parts; ++p) off[p + 1] = off[p] + pid[p].size();
  out.ids.resize(off[parts]);
  out.levcnt.resize(8 * off[parts]);
  parallel_dyn(T, parts, 8, [&](int, int64_t p) {
    if (pid[p].empty()) return;
    std::memcpy(out.ids.data() + off[p], pid[p].data(), 4 * pid[p].size());
    std::memcpy(out.levcnt.data() + 8 * off[p], plev[p].data(), 8 * plev[p].size());
  });
}

// est_v = (1/M) Σ_l N1 D^(l-1) levcnt[v][l]  (eq. (3) averaged over M walks)
double estimate_value(const uint64_t *lev, int k, uint64_t N1, uint64_t D, uint64_t M) {
  double e = 0.0;
  for (int l = 1; l <= k - 2; ++l) e += (double)N1 * std::pow((double)D, (double)(l - 1)) * (double)lev[l - 1];
  return e / (double)M;
}

}  // namespace gcsm
