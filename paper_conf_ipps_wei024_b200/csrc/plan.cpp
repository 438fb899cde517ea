// plan.cpp — query plan builder (IVM terms of eq. (1) as the nested loops of Fig. 2b-f).
//
// PAPER.md P:125-136 (eq. (1)): with the query edges numbered R_1..R_m,
//   ΔM_i = R_1 ⋈ … ⋈ R_{i-1} ⋈ ΔR_i ⋈ R'_{i+1} ⋈ … ⋈ R'_m.
// P:142 / Fig. 2b-f: term i iterates the updated edges matching
// R_i and extends the remaining query vertices by set intersections.
// Readings:
//   R12 numbering: lexicographic by (min, max) position in the user order (Fig. 2);
//   R11 term order: the seed endpoints, then repeatedly the first vertex of the
//       user order adjacent to the placed set (ΔM_4 = u1,u3,u0,u2);
//   R7  views ("stable split"): j < i reads the stable lists S = E ∩ E';
//       j > i reads N' (insertion terms) or N (deletion terms) — exact per-sign
//       added/removed counts, whose difference is eq. (1)'s net.
// Code motion (STMatch [9]): a later position whose lists contain an
// earlier position's lists (same views, same label) starts from that
// position's candidate set instead of re-intersecting.
#include <algorithm>
#include <cstring>
#include <numeric>

#include "internal.h"

namespace gcsm {

static View view_for(int j, int term, int kind) {
  if (j < term) return VIEW_S;
  return kind == 0 ? VIEW_NEW : VIEW_OLD;
}

std::string build_plan(int k, int m, const int32_t *qedges, const int32_t *qlabels, const int32_t *order,
                       QueryPlan &out, bool symmetry) {
  if (k < 2 || k > GCSM_MAXK) return "query size k must be in [2, 8]";
  if (m < 1 || m > k * (k - 1) / 2) return "query edge count m out of range";
  if (!qedges) return "qedges is NULL";
  bool adj[GCSM_MAXK][GCSM_MAXK] = {};
  for (int i = 0; i < m; ++i) {
    int u = qedges[2 * i], w = qedges[2 * i + 1];
    if (u < 0 || w < 0 || u >= k || w >= k) return "query edge endpoint out of range";
    if (u == w) return "query self loop";
    if (adj[u][w]) return "duplicate query edge";
    adj[u][w] = adj[w][u] = true;
  }
  {  // connected
    int seen = 1, stack[GCSM_MAXK], sp = 0;
    bool vis[GCSM_MAXK] = {};
    vis[0] = true;
    stack[sp++] = 0;
    while (sp) {
      int u = stack[--sp];
      for (int w = 0; w < k; ++w)
        if (adj[u][w] && !vis[w]) { vis[w] = true; ++seen; stack[sp++] = w; }
    }
    if (seen != k) return "query is not connected";
  }
  int uo[GCSM_MAXK], pos[GCSM_MAXK];
  for (int i = 0; i < k; ++i) pos[i] = -1;
  for (int i = 0; i < k; ++i) {
    uo[i] = order ? order[i] : i;
    if (uo[i] < 0 || uo[i] >= k || pos[uo[i]] >= 0) return "order is not a permutation of [0,k)";
    pos[uo[i]] = i;
  }
  QueryPlan q;
  q.k = k;
  q.m = m;
  q.labelled = qlabels != nullptr;
  for (int u = 0; u < k; ++u) {
    q.qlab[u] = qlabels ? qlabels[u] : -1;
    if (qlabels && (qlabels[u] < 0 || qlabels[u] > 65535)) return "query label out of [0, 65535]";
  }
  // R12: number the query edges by (min position, max position)
  std::vector<std::pair<int, int>> e(m);
  for (int i = 0; i < m; ++i) {
    int u = qedges[2 * i], w = qedges[2 * i + 1];
    if (pos[u] > pos[w]) std::swap(u, w);
    e[i] = {u, w};
  }
  std::sort(e.begin(), e.end(), [&](const std::pair<int, int> &x, const std::pair<int, int> &y) {
    return std::make_pair(pos[x.first], pos[x.second]) < std::make_pair(pos[y.first], pos[y.second]);
  });
  int eidx[GCSM_MAXK][GCSM_MAXK];
  for (int i = 0; i < m; ++i) {
    q.qe[i][0] = e[i].first;
    q.qe[i][1] = e[i].second;
    eidx[e[i].first][e[i].second] = eidx[e[i].second][e[i].first] = i;
  }
  // automorphisms (label preserving)
  std::vector<std::vector<int>> auts;
  {
    int p[GCSM_MAXK];
    std::iota(p, p + k, 0);
    do {
      bool ok = true;
      for (int u = 0; u < k && ok; ++u)
        if (q.qlab[p[u]] != q.qlab[u]) ok = false;
      for (int i = 0; i < m && ok; ++i)
        if (!adj[p[q.qe[i][0]]][p[q.qe[i][1]]]) ok = false;
      if (ok) auts.emplace_back(p, p + k);
    } while (std::next_permutation(p, p + k));
    q.automorphisms = auts.size();
  }
  // Symmetry breaking (Grochow & Kellis): walk the user order; for the first vertex v with a non-trivial orbit
  // under the current group require f(v) < f(w) for the rest of its orbit, then keep only v's stabiliser.
  // Exactly one embedding of every Aut_L orbit {f o s} satisfies all restrictions (pinned by brute force in
  // tests/test_abi.py), and Emb(G') \ Emb(G) is a union of orbits, so counts = |Aut_L| x restricted counts.
  q.symmetry = symmetry && auts.size() > 1;
  if (q.symmetry) {
    std::vector<std::vector<int>> G = auts;
    for (int r = 0; r < k && G.size() > 1; ++r) {
      const int v = uo[r];
      bool seen[GCSM_MAXK] = {};
      for (const auto &p : G) seen[p[v]] = true;
      for (int w = 0; w < k; ++w)
        if (seen[w] && w != v) q.restrictions.push_back({v, w});
      std::vector<std::vector<int>> H;
      for (const auto &p : G)
        if (p[v] == v) H.push_back(p);
      G.swap(H);
    }
  }
  q.plans.resize(2 * m);
  for (int term = 0; term < m; ++term) {
    // R11: term order
    int ord[GCSM_MAXK], n = 0;
    bool placed[GCSM_MAXK] = {};
    ord[n++] = q.qe[term][0];
    ord[n++] = q.qe[term][1];
    placed[ord[0]] = placed[ord[1]] = true;
    while (n < k) {
      for (int r = 0; r < k; ++r) {
        int z = uo[r];
        if (placed[z]) continue;
        bool touch = false;
        for (int s = 0; s < n; ++s) touch |= adj[ord[s]][z];
        if (touch) { ord[n++] = z; placed[z] = true; break; }
      }
    }
    for (int kind = 0; kind < 2; ++kind) {
      DevPlan &P = q.plans[2 * term + kind];
      std::memset(&P, 0, sizeof P);
      P.k = k;
      P.kind = kind;
      for (int s = 0; s < k; ++s) P.order[s] = (int8_t)ord[s];
      P.label0 = q.qlab[ord[0]];
      P.label1 = q.qlab[ord[1]];
      int posof[GCSM_MAXK];
      for (int s2 = 0; s2 < k; ++s2) posof[ord[s2]] = s2;
      P.seed_rel = 0;
      for (const auto &rw : q.restrictions) {
        const int pu = posof[rw.first], pw = posof[rw.second];  // f(order[pu]) < f(order[pw])
        if (std::max(pu, pw) == 1) {
          P.seed_rel = pu == 0 ? 1 : 2;
        } else if (pw > pu) {  // placed at pw: must exceed f at pu
          LevelPlan &L = P.lv[pw];
          L.lo[L.nlo++] = (int8_t)pu;
        } else {  // placed at pu: must stay below f at pw
          LevelPlan &L = P.lv[pu];
          L.hi[L.nhi++] = (int8_t)pw;
        }
      }
      for (int p = 2; p < k; ++p) {
        LevelPlan &L = P.lv[p];
        L.label = q.qlab[ord[p]];
        L.reuse = -1;
        bool back[GCSM_MAXK] = {};
        for (int s = 0; s < p; ++s) {
          if (!adj[ord[s]][ord[p]]) continue;
          L.bpos[L.nb] = (int8_t)s;
          L.bview[L.nb] = (int8_t)view_for(eidx[ord[s]][ord[p]], term, kind);
          L.nb++;
          back[s] = true;
        }
        for (int s = 0; s < p; ++s)
          if (!back[s]) L.inj[L.ninj++] = (int8_t)s;
        // code motion: latest earlier position p' >= 2 with the same label whose lists ⊆ ours
        for (int pp = p - 1; pp >= 2 && L.reuse < 0; --pp) {
          const LevelPlan &E = P.lv[pp];
          if (E.label != L.label) continue;
          // the earlier set was filtered by its own symmetry restrictions: they must bind here too
          bool implied = true;
          for (int a = 0; a < E.nlo && implied; ++a) {
            bool f = false;
            for (int b = 0; b < L.nlo; ++b) f |= E.lo[a] == L.lo[b];
            implied = f;
          }
          for (int a = 0; a < E.nhi && implied; ++a) {
            bool f = false;
            for (int b = 0; b < L.nhi; ++b) f |= E.hi[a] == L.hi[b];
            implied = f;
          }
          if (!implied) continue;
          bool sub = true;
          for (int a = 0; a < E.nb && sub; ++a) {
            bool found = false;
            for (int b = 0; b < L.nb; ++b) found |= (E.bpos[a] == L.bpos[b] && E.bview[a] == L.bview[b]);
            sub = found;
          }
          if (!sub) continue;
          L.reuse = (int8_t)pp;
          L.nrest = 0;
          for (int b = 0; b < L.nb; ++b) {
            bool covered = false;
            for (int a = 0; a < E.nb; ++a) covered |= (E.bpos[a] == L.bpos[b] && E.bview[a] == L.bview[b]);
            if (!covered) L.rest[L.nrest++] = (int8_t)b;
          }
        }
        // loop-invariant code motion of the last level (k >= 5): the lists of backward positions <= 2 are fixed
        // for a whole level-2 entry; with >= 2 of them their intersection is computed once per entry
        // level-3 filter (k >= 5): position 4's lists at positions <= 2 against each level-3 node's own list
        L.fmask = 0;
        L.f3 = -1;
        if (p == 4 && k >= 6) {  // (k = 5: position 4 is the last one, where the filter test IS the count: C3 10.9 vs 18.8 ms per step, profiles/ab8_r02.txt)
          int msk = 0, b3 = -1;
          for (int b = 0; b < L.nb; ++b) {
            if (L.bpos[b] <= 2) msk |= 1 << b;
            if (L.bpos[b] == 3) b3 = b;
          }
          if (b3 >= 0 && msk) {
            L.fmask = (int8_t)msk;
            L.f3 = (int8_t)b3;
          }
        }
        L.hmask = 0;
        if (p == k - 1 && k >= 5 && L.reuse < 0) {
          int cnt = 0, msk = 0;
          for (int b = 0; b < L.nb; ++b)
            if (L.bpos[b] <= 2) {
              msk |= 1 << b;
              ++cnt;
            }
          if (cnt >= 2) L.hmask = (int8_t)msk;
        }
      }

    }
  }
  out = q;
  return "";
}

// Greedy LPT: units by cost descending (ties: lower index first) each go to
// the least-loaded rank (ties: lower rank). Deterministic on every rank.
// The descending order is a parallel stable sort (the same order as a serial one); *order_out (optional) receives
// it, so a caller can keep its own units heaviest first without sorting again.
void shard_lpt(int64_t n, const uint64_t *cost, int world, int32_t *rank_out, int threads,
               std::vector<size_t> *order_out) {
  std::vector<size_t> idx((size_t)n);
  std::iota(idx.begin(), idx.end(), 0);
  if (world > 1 || order_out)
    parallel_sort(idx, [&](size_t x, size_t y) { return cost[x] > cost[y]; }, std::max(1, threads), /*stable=*/true);
  std::vector<uint64_t> load(std::max(1, world), 0);
  for (int64_t t = 0; t < n; ++t) {
    int best = 0;
    for (int r = 1; r < world; ++r)
      if (load[r] < load[best]) best = r;
    rank_out[idx[t]] = best;
    load[best] += cost[idx[t]] + 1;
  }
  if (order_out) order_out->swap(idx);
}

}  // namespace gcsm
