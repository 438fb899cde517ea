/*
 * oracle/oracle.c — TEST INFRASTRUCTURE ONLY (never part of the product path).
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * `--impl reference` legs may load or execute this file's library. It shares
 * no code, header, table or helper with paper_conf_ipps_wei024_b200/ and
 * never imports it.
 *
 * A plain, slow, obviously-correct CPU implementation of what the GCSM hot
 * path computes (PAPER.md = "P:<line>"):
 *
 *  o3_delta    — the DEFINITION of the batch delta:
 *                embeddings of Q in a graph that use >= 1 changed edge, each
 *                counted once (attributed to its minimum changed data edge).
 *                added = o3_delta(G_{t+1}, I), removed = o3_delta(G_t, D).
 *  o2_static   — all embeddings of Q in G (static recount; telescoping pin).
 *  ivm_*       — the ALGORITHM of the paper in its own order: the IVM delta
 *                terms of eq. (1) run as the nested loops of
 *                Fig. 2b-f with the stable-split views of
 *                DESIGN.md reading R7; used for
 *                  * its counts (must equal o3_delta: pins reading R7),
 *                  * exact per-vertex access counts C_v (Fig. 15),
 *                  * M plain random walks of §IV-A, one at a
 *                    time, exactly as the paper states them (pick a unit
 *                    with probability 1/|ΔE|, a child with 1/|V|, continue
 *                    with |V|/D), drawn from the oracle's own PCG32 streams;
 *                    eq. (3) weighs what they record. The paper's
 *                    merged form (§IV-B, binomial multiplicities) is the
 *                    product's business and is NOT reproduced here.
 *
 * Match semantics (readings R1-R5): non-induced, injective,
 * vertex-labelled embeddings of an undirected simple query graph.
 */
#include <math.h>
#include <pthread.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define OMAXK 8
#define OMAXM 28

typedef unsigned __int128 u128;

typedef struct {
  int32_t n;
  const int64_t *rp;
  const int32_t *col;
} ograph;

typedef struct {
  int k, m;
  int e[OMAXM][2];
  const int32_t *qlab; /* NULL = unlabelled */
  int adj[OMAXK][OMAXK];
} oquery;

static int row_has(const ograph *g, int32_t u, int32_t v) {
  int64_t lo = g->rp[u], hi = g->rp[u + 1];
  while (lo < hi) {
    int64_t mid = lo + (hi - lo) / 2;
    if (g->col[mid] < v) lo = mid + 1;
    else hi = mid;
  }
  return lo < g->rp[u + 1] && g->col[lo] == v;
}

static uint64_t ekey(int32_t a, int32_t b) {
  if (a > b) { int32_t t = a; a = b; b = t; }
  return ((uint64_t)(uint32_t)a << 32) | (uint32_t)b;
}

static int key_in(const uint64_t *keys, int64_t n, uint64_t key) {
  int64_t lo = 0, hi = n;
  while (lo < hi) {
    int64_t mid = lo + (hi - lo) / 2;
    if (keys[mid] < key) lo = mid + 1;
    else hi = mid;
  }
  return lo < n && keys[lo] == key;
}

static int query_init(oquery *q, int k, int m, const int32_t *qe, const int32_t *ql) {
  if (k < 2 || k > OMAXK || m < 1 || m > OMAXM) return -1;
  q->k = k;
  q->m = m;
  q->qlab = ql;
  memset(q->adj, 0, sizeof q->adj);
  for (int i = 0; i < m; ++i) {
    q->e[i][0] = qe[2 * i];
    q->e[i][1] = qe[2 * i + 1];
    q->adj[qe[2 * i]][qe[2 * i + 1]] = q->adj[qe[2 * i + 1]][qe[2 * i]] = 1;
  }
  return 0;
}

static int label_ok(const int32_t *lab, const oquery *q, int u, int32_t v) {
  if (!q->qlab) return 1;
  return (lab ? lab[v] : 0) == q->qlab[u];
}

/* ------------------------------------------------------------------ work pool */

typedef struct {
  int64_t n_items;
  int64_t next;
  pthread_mutex_t mu;
  void *(*fn)(void *);
} pool_t;

static int64_t pool_take(pool_t *p) {
  pthread_mutex_lock(&p->mu);
  int64_t i = p->next < p->n_items ? p->next++ : -1;
  pthread_mutex_unlock(&p->mu);
  return i;
}

static void run_threads(int threads, void *(*fn)(void *), void **args) {
  pthread_t th[256];
  if (threads < 1) threads = 1;
  if (threads > 256) threads = 256;
  for (int t = 0; t < threads; ++t) pthread_create(&th[t], NULL, fn, args[t]);
  for (int t = 0; t < threads; ++t) pthread_join(th[t], NULL);
}

/* ================================================================== graph update */
/*
 * G_{t+1} = (E \ D) ∪ I row by row (reading R8): for every vertex,
 * its list minus the deleted neighbours plus the inserted ones, sorted.
 * ins/del: canonical pairs already normalised (I ∩ E = ∅, D ⊆ E). The caller
 * sizes out_col as rp[n] + 2|I| - 2|D|.
 */
static int cmp_i32(const void *a, const void *b) {
  int32_t x = *(const int32_t *)a, y = *(const int32_t *)b;
  return x < y ? -1 : x > y;
}

int o_apply(int32_t n, const int64_t *rp, const int32_t *col, int64_t n_ins, const int32_t *ins, int64_t n_del,
            const int32_t *del, int64_t *out_rp, int32_t *out_col) {
  /* per-vertex change lists */
  int64_t *ci = (int64_t *)calloc((size_t)n + 1, sizeof(int64_t));
  int64_t *cd = (int64_t *)calloc((size_t)n + 1, sizeof(int64_t));
  for (int64_t e = 0; e < n_ins; ++e) { ci[ins[2 * e] + 1]++; ci[ins[2 * e + 1] + 1]++; }
  for (int64_t e = 0; e < n_del; ++e) { cd[del[2 * e] + 1]++; cd[del[2 * e + 1] + 1]++; }
  for (int32_t v = 0; v < n; ++v) { ci[v + 1] += ci[v]; cd[v + 1] += cd[v]; }
  int32_t *vi = (int32_t *)malloc(sizeof(int32_t) * (size_t)(2 * n_ins + 1));
  int32_t *vd = (int32_t *)malloc(sizeof(int32_t) * (size_t)(2 * n_del + 1));
  int64_t *pi = (int64_t *)malloc(sizeof(int64_t) * ((size_t)n + 1));
  int64_t *pd = (int64_t *)malloc(sizeof(int64_t) * ((size_t)n + 1));
  memcpy(pi, ci, sizeof(int64_t) * ((size_t)n + 1));
  memcpy(pd, cd, sizeof(int64_t) * ((size_t)n + 1));
  for (int64_t e = 0; e < n_ins; ++e) { vi[pi[ins[2 * e]]++] = ins[2 * e + 1]; vi[pi[ins[2 * e + 1]]++] = ins[2 * e]; }
  for (int64_t e = 0; e < n_del; ++e) { vd[pd[del[2 * e]]++] = del[2 * e + 1]; vd[pd[del[2 * e + 1]]++] = del[2 * e]; }
  out_rp[0] = 0;
  for (int32_t v = 0; v < n; ++v) {
    int64_t w = out_rp[v];
    for (int64_t e = rp[v]; e < rp[v + 1]; ++e) {
      int gone = 0;
      for (int64_t j = cd[v]; j < cd[v + 1]; ++j) if (vd[j] == col[e]) gone = 1;
      if (!gone) out_col[w++] = col[e];
    }
    for (int64_t j = ci[v]; j < ci[v + 1]; ++j) out_col[w++] = vi[j];
    qsort(out_col + out_rp[v], (size_t)(w - out_rp[v]), sizeof(int32_t), cmp_i32);
    out_rp[v + 1] = w;
  }
  free(ci); free(cd); free(vi); free(vd); free(pi); free(pd);
  return 0;
}

/* ================================================================== O3 / O2 */
/*
 * Plain backtracking: positions `ord[0..k-1]` (a BFS order of Q from the seed
 * query edge), f[u] = data vertex of query vertex u. A vertex is extended from
 * the adjacency of one matched query neighbour, then every query edge to the
 * matched set is checked by binary search; labels and injectivity are checked.
 */
typedef struct {
  const ograph *g;
  const int32_t *lab;
  const oquery *q;
  const uint64_t *chg; /* sorted canonical keys of changed edges (O3) */
  int64_t n_chg;
  int ord[OMAXK];
  int par[OMAXK]; /* a matched query neighbour of ord[p] (p >= 1) */
  int32_t f[OMAXK];
  uint64_t seed_key;
  u128 count;
  /* listing (single-thread only) */
  int32_t *tuples;
  int64_t tuple_cap, n_tuples;
} bt_t;

static void bfs_order(const oquery *q, int s0, int s1, int *ord, int *par) {
  int placed[OMAXK] = {0};
  int n = 0;
  ord[n] = s0; par[n++] = -1; placed[s0] = 1;
  if (s1 >= 0) { ord[n] = s1; par[n++] = s0; placed[s1] = 1; }
  for (int h = 0; h < n && n < q->k; ++h)
    for (int z = 0; z < q->k; ++z)
      if (!placed[z] && q->adj[ord[h]][z]) { ord[n] = z; par[n++] = ord[h]; placed[z] = 1; }
}

static void bt_emit(bt_t *s) {
  if (s->chg) {
    /* count f only if the seed edge is the minimum changed edge it uses */
    uint64_t mn = UINT64_MAX;
    for (int i = 0; i < s->q->m; ++i) {
      uint64_t key = ekey(s->f[s->q->e[i][0]], s->f[s->q->e[i][1]]);
      if (key < mn && key_in(s->chg, s->n_chg, key)) mn = key;
    }
    if (mn != s->seed_key) return;
  }
  s->count += 1;
  if (s->tuples) {
    if (s->n_tuples < s->tuple_cap)
      for (int u = 0; u < s->q->k; ++u) s->tuples[s->n_tuples * s->q->k + u] = s->f[u];
    s->n_tuples++;
  }
}

static void bt_rec(bt_t *s, int p) {
  if (p == s->q->k) { bt_emit(s); return; }
  const int z = s->ord[p];
  const int32_t src = s->f[s->par[p]];
  for (int64_t e = s->g->rp[src]; e < s->g->rp[src + 1]; ++e) {
    const int32_t c = s->g->col[e];
    if (!label_ok(s->lab, s->q, z, c)) continue;
    int ok = 1;
    for (int t = 0; t < p && ok; ++t) if (s->f[s->ord[t]] == c) ok = 0;
    for (int t = 0; t < p && ok; ++t)
      if (s->q->adj[s->ord[t]][z] && !row_has(s->g, s->f[s->ord[t]], c)) ok = 0;
    if (!ok) continue;
    s->f[z] = c;
    bt_rec(s, p + 1);
  }
}

typedef struct {
  pool_t *pool;
  const ograph *g;
  const int32_t *lab;
  const oquery *q;
  const int32_t *chg_pairs;
  const uint64_t *chg_keys;
  int64_t n_chg;
  u128 count;
  int32_t *tuples;
  int64_t tuple_cap, n_tuples;
} o3_arg;

/* item = (changed edge index, query edge index, orientation) */
static void o3_item(o3_arg *a, bt_t *s, int64_t it) {
  const int64_t ei = it / (2 * a->q->m);
  const int qi = (int)((it / 2) % a->q->m);
  const int o = (int)(it % 2);
  int32_t x = a->chg_pairs[2 * ei], y = a->chg_pairs[2 * ei + 1];
  if (o) { int32_t t = x; x = y; y = t; }
  const int u = a->q->e[qi][0], w = a->q->e[qi][1];
  if (!label_ok(a->lab, a->q, u, x) || !label_ok(a->lab, a->q, w, y)) return;
  if (!row_has(a->g, x, y)) return; /* changed edge must exist in this graph */
  bfs_order(a->q, u, w, s->ord, s->par);
  s->f[u] = x;
  s->f[w] = y;
  s->seed_key = ekey(x, y);
  bt_rec(s, 2);
}

static void *o3_worker(void *vp) {
  o3_arg *a = (o3_arg *)vp;
  bt_t s;
  memset(&s, 0, sizeof s);
  s.g = a->g; s.lab = a->lab; s.q = a->q; s.chg = a->chg_keys; s.n_chg = a->n_chg;
  s.tuples = a->tuples; s.tuple_cap = a->tuple_cap;
  for (int64_t it; (it = pool_take(a->pool)) >= 0;) o3_item(a, &s, it);
  a->count = s.count;
  a->n_tuples = s.n_tuples;
  return NULL;
}

static int cmp_u64(const void *a, const void *b) {
  uint64_t x = *(const uint64_t *)a, y = *(const uint64_t *)b;
  return x < y ? -1 : x > y;
}

/*
 * Number of embeddings of Q in graph (n,rp,col) that map >= 1 query edge onto
 * one of the n_chg changed edges (chg: canonical pairs, all present in the
 * graph). out[0..1] = low/high 64 bits of the exact count. Listing: if tuples
 * != NULL, runs single-threaded and writes up to tuple_cap k-tuples (query
 * vertex order); *n_tuples = the total number found.
 */
int o3_delta(int32_t n, const int64_t *rp, const int32_t *col, const int32_t *lab, int32_t k, int32_t m,
             const int32_t *qe, const int32_t *ql, int64_t n_chg, const int32_t *chg, int32_t threads,
             uint64_t *out, int32_t *tuples, int64_t tuple_cap, int64_t *n_tuples) {
  oquery q;
  if (query_init(&q, k, m, qe, ql)) return -1;
  ograph g = {n, rp, col};
  uint64_t *keys = (uint64_t *)malloc(sizeof(uint64_t) * (size_t)(n_chg > 0 ? n_chg : 1));
  for (int64_t i = 0; i < n_chg; ++i) keys[i] = ekey(chg[2 * i], chg[2 * i + 1]);
  qsort(keys, (size_t)n_chg, sizeof(uint64_t), cmp_u64);
  pool_t pool = {n_chg * 2 * m, 0, PTHREAD_MUTEX_INITIALIZER, NULL};
  if (tuples) threads = 1;
  if (threads < 1) threads = 1;
  o3_arg *args = (o3_arg *)calloc((size_t)threads, sizeof(o3_arg));
  void *ptrs[256];
  for (int t = 0; t < threads && t < 256; ++t) {
    args[t] = (o3_arg){&pool, &g, lab, &q, chg, keys, n_chg, 0, tuples, tuple_cap, 0};
    ptrs[t] = &args[t];
  }
  run_threads(threads, o3_worker, ptrs);
  u128 tot = 0;
  int64_t nt = 0;
  for (int t = 0; t < threads && t < 256; ++t) { tot += args[t].count; nt += args[t].n_tuples; }
  out[0] = (uint64_t)tot;
  out[1] = (uint64_t)(tot >> 64);
  if (n_tuples) *n_tuples = nt;
  free(args);
  free(keys);
  return 0;
}

typedef struct {
  pool_t *pool;
  const ograph *g;
  const int32_t *lab;
  const oquery *q;
  u128 count;
} o2_arg;

static void *o2_worker(void *vp) {
  o2_arg *a = (o2_arg *)vp;
  bt_t s;
  memset(&s, 0, sizeof s);
  s.g = a->g; s.lab = a->lab; s.q = a->q;
  bfs_order(a->q, 0, -1, s.ord, s.par);
  for (int64_t v; (v = pool_take(a->pool)) >= 0;) {
    if (!label_ok(a->lab, a->q, 0, (int32_t)v)) continue;
    s.f[0] = (int32_t)v;
    bt_rec(&s, 1);
  }
  a->count = s.count;
  return NULL;
}

/* |Emb(Q, G)| for a connected query (static recount). */
int o2_static(int32_t n, const int64_t *rp, const int32_t *col, const int32_t *lab, int32_t k, int32_t m,
              const int32_t *qe, const int32_t *ql, int32_t threads, uint64_t *out) {
  oquery q;
  if (query_init(&q, k, m, qe, ql)) return -1;
  ograph g = {n, rp, col};
  pool_t pool = {n, 0, PTHREAD_MUTEX_INITIALIZER, NULL};
  if (threads < 1) threads = 1;
  o2_arg *args = (o2_arg *)calloc((size_t)threads, sizeof(o2_arg));
  void *ptrs[256];
  for (int t = 0; t < threads && t < 256; ++t) { args[t] = (o2_arg){&pool, &g, lab, &q, 0}; ptrs[t] = &args[t]; }
  run_threads(threads, o2_worker, ptrs);
  u128 tot = 0;
  for (int t = 0; t < threads && t < 256; ++t) tot += args[t].count;
  out[0] = (uint64_t)tot;
  out[1] = (uint64_t)(tot >> 64);
  free(args);
  return 0;
}

/* ================================================================== IVM terms */
/*
 * Term plans (readings R11, R12, R7):
 *  - query edges are numbered R_1..R_m lexicographically by
 *    (min position, max position) in the user order (Fig. 2 numbering);
 *  - term i seeds query edge e_i = (u_x, u_y), pos(u_x) < pos(u_y); its order is
 *    u_x, u_y, then repeatedly the first vertex of the user order adjacent to
 *    the placed set (Fig. 2b-f);
 *  - the backward edge (u_q, z) with edge index j is read through view
 *      STABLE if j < i; NEW (+ term) / OLD (- term) if j > i.
 */
enum { V_STABLE = 0, V_OLD = 1, V_NEW = 2 };

typedef struct {
  int order[OMAXK];
  int nb[OMAXK];          /* number of backward edges of position p */
  int bq[OMAXK][OMAXK];   /* backward positions */
  int bj[OMAXK][OMAXK];   /* edge index of each backward edge */
} oterm;

static void number_edges(const oquery *q, const int *user_order, int *eidx_of /* m */, int (*num)[2]) {
  int pos[OMAXK];
  for (int i = 0; i < q->k; ++i) pos[user_order[i]] = i;
  int keyv[OMAXM], idx[OMAXM];
  for (int i = 0; i < q->m; ++i) {
    int a = pos[q->e[i][0]], b = pos[q->e[i][1]];
    if (a > b) { int t = a; a = b; b = t; }
    keyv[i] = a * OMAXK + b;
    idx[i] = i;
  }
  for (int i = 0; i < q->m; ++i) /* insertion sort by key */
    for (int j = i; j > 0 && keyv[idx[j]] < keyv[idx[j - 1]]; --j) { int t = idx[j]; idx[j] = idx[j - 1]; idx[j - 1] = t; }
  for (int r = 0; r < q->m; ++r) {
    int i = idx[r];
    int a = q->e[i][0], b = q->e[i][1];
    if (pos[a] > pos[b]) { int t = a; a = b; b = t; }
    num[r][0] = a; num[r][1] = b;
    eidx_of[i] = r;
  }
}

static void build_term(const oquery *q, const int *user_order, int (*num)[2], int i, oterm *t) {
  int placed[OMAXK] = {0};
  int n = 0;
  t->order[n++] = num[i][0]; placed[num[i][0]] = 1;
  t->order[n++] = num[i][1]; placed[num[i][1]] = 1;
  while (n < q->k) {
    for (int r = 0; r < q->k; ++r) {
      int z = user_order[r];
      if (placed[z]) continue;
      int adj = 0;
      for (int p = 0; p < n; ++p) adj |= q->adj[t->order[p]][z];
      if (adj) { t->order[n++] = z; placed[z] = 1; break; }
    }
  }
  for (int p = 0; p < q->k; ++p) {
    t->nb[p] = 0;
    if (p < 2) continue;
    for (int s = 0; s < p; ++s) {
      int a = t->order[s], z = t->order[p];
      if (!q->adj[a][z]) continue;
      int j = -1;
      for (int r = 0; r < q->m; ++r)
        if ((num[r][0] == a && num[r][1] == z) || (num[r][0] == z && num[r][1] == a)) j = r;
      t->bq[p][t->nb[p]] = s;
      t->bj[p][t->nb[p]] = j;
      t->nb[p]++;
    }
  }
}

static int view_of(int j, int i, int kind /*0 = +, 1 = -*/) {
  if (j < i) return V_STABLE;
  return kind == 0 ? V_NEW : V_OLD;
}

/*
 * Exported for the plan structural test (SURVEY §4 table vs Fig. 2):
 * out_order[m*k], out_nb[m*k], out_bq[m*k*8], out_view[2*m*k*8] (kind-major),
 * out_seed[2m] (numbered query edges).
 */
int ivm_plan(int32_t k, int32_t m, const int32_t *qe, const int32_t *user_order, int32_t *out_order, int32_t *out_nb,
             int32_t *out_bq, int32_t *out_view, int32_t *out_seed) {
  oquery q;
  if (query_init(&q, k, m, qe, NULL)) return -1;
  int uo[OMAXK], num[OMAXM][2], eidx[OMAXM];
  for (int i = 0; i < k; ++i) uo[i] = user_order ? user_order[i] : i;
  number_edges(&q, uo, eidx, num);
  for (int i = 0; i < m; ++i) {
    oterm t;
    build_term(&q, uo, num, i, &t);
    out_seed[2 * i] = num[i][0];
    out_seed[2 * i + 1] = num[i][1];
    for (int p = 0; p < k; ++p) {
      out_order[i * k + p] = t.order[p];
      out_nb[i * k + p] = t.nb[p];
      for (int b = 0; b < t.nb[p]; ++b) {
        out_bq[(i * k + p) * 8 + b] = t.bq[p][b];
        for (int kind = 0; kind < 2; ++kind)
          out_view[((kind * m + i) * k + p) * 8 + b] = view_of(t.bj[p][b], i, kind);
      }
    }
  }
  return 0;
}

/* ---------------------------------------------------------- the nested loops */
typedef struct {
  const ograph *g[3]; /* indexed by view: STABLE, OLD, NEW */
  const int32_t *lab;
  const oquery *q;
  oterm terms[OMAXM];
  int mode; /* 0 count, 1 access, 2 plain random walks */
  /* walks */
  uint64_t seed;
  int64_t M, N1, D;
  /* outputs (shared; atomics) */
  uint64_t *access;  /* n (mode 1) */
  uint64_t *levcnt;  /* n * (k-2) (mode 2) */
  /* units */
  int64_t n_units;
  const int32_t *units; /* [n_units][4]: term, kind, a, b */
} ivm_ctx;

typedef struct {
  const ivm_ctx *c;
  const oterm *t;
  int kind;
  int32_t f[OMAXK]; /* by term position */
  u128 count;
} ivm_state;

/* Candidates for term position p: elements of the first backward list present
 * in every other backward list, with the query label of order[p] and not
 * equal to any matched vertex. Returns the number written to out. */
static int64_t ivm_candidates(ivm_state *s, int p, int32_t *out) {
  const oterm *t = s->t;
  const ivm_ctx *c = s->c;
  const int z = t->order[p];
  const ograph *g0 = c->g[view_of(t->bj[p][0], (int)(t - c->terms), s->kind)];
  const int32_t x0 = s->f[t->bq[p][0]];
  int64_t n = 0;
  for (int64_t e = g0->rp[x0]; e < g0->rp[x0 + 1]; ++e) {
    const int32_t v = g0->col[e];
    int ok = label_ok(c->lab, c->q, z, v);
    for (int s2 = 0; s2 < p && ok; ++s2) if (s->f[s2] == v) ok = 0;
    for (int b = 1; b < t->nb[p] && ok; ++b) {
      const ograph *gb = c->g[view_of(t->bj[p][b], (int)(t - c->terms), s->kind)];
      if (!row_has(gb, s->f[t->bq[p][b]], v)) ok = 0;
    }
    if (ok) out[n++] = v;
  }
  return n;
}

static void ivm_visit(ivm_state *s, int level) {
  /* node at `level` has positions 0..level matched; it computes position level+1 */
  const int k = s->c->q->k;
  if (level >= k - 1) { s->count += 1; return; } /* leaf: a complete embedding */
  const int p = level + 1;
  const oterm *t = s->t;
  if (s->c->mode == 1)
    for (int b = 0; b < t->nb[p]; ++b) __atomic_fetch_add(&s->c->access[s->f[t->bq[p][b]]], 1, __ATOMIC_RELAXED);
  int32_t *cand = (int32_t *)malloc(sizeof(int32_t) * (size_t)(s->c->D + 1));
  const int64_t nc = ivm_candidates(s, p, cand);
  for (int64_t i = 0; i < nc; ++i) {
    s->f[p] = cand[i];
    ivm_visit(s, level + 1);
  }
  free(cand);
}

/* ---------------------------------------------------------- plain random walks (§IV-A) */
/* The oracle's own generator: PCG32 (O'Neill 2014, XSH-RR 64/32), one stream per walk index, so the result is
 * the same for any thread count. The paper fixes no RNG; this one shares nothing with the product's. */
typedef struct { uint64_t state, inc; } opcg;
static uint32_t opcg_next(opcg *r) {
  const uint64_t old = r->state;
  r->state = old * 6364136223846793005ULL + r->inc;
  const uint32_t xs = (uint32_t)(((old >> 18) ^ old) >> 27), rot = (uint32_t)(old >> 59);
  return (xs >> rot) | (xs << ((32u - rot) & 31u));
}
static void opcg_seed(opcg *r, uint64_t initstate, uint64_t stream) {
  r->state = 0;
  r->inc = (stream << 1) | 1u;
  opcg_next(r);
  r->state += initstate;
  opcg_next(r);
}
/* uniform integer in [0, n), n >= 1, by rejection of the top partial block of 2^64 */
static uint64_t opcg_below(opcg *r, uint64_t n) {
  const uint64_t lim = UINT64_MAX - UINT64_MAX % n;
  for (;;) {
    const uint64_t x = ((uint64_t)opcg_next(r) << 32) | opcg_next(r);
    if (x < lim) return x % n;
  }
}

/* One random walk of §IV-A: "randomly select one edge from ΔE, with a probability of 1/|ΔE|" (here one level-1
 * unit of the forest of all terms, R15/R16); "compute the set of matching vertices V for the next pattern
 * vertex", "randomly select one vertex from V, with a probability of 1/|V|", then "continue the walk with a
 * probability of |V|/D". Each node on the path records the lists it accesses (R17: the backward lists of the
 * next position; leaves access nothing): levcnt[v][l-1] counts the walk's level-l node reading v's list, and
 * eq. (3) weighs it by |ΔE| D^(l-1) (done in Python). */
static void ow_walk(const ivm_ctx *c, int64_t w, int32_t *cand) {
  opcg r;
  opcg_seed(&r, c->seed, (uint64_t)w);
  const int k = c->q->k;
  const int32_t *un = c->units + 4 * (int64_t)opcg_below(&r, (uint64_t)c->N1);
  ivm_state s;
  memset(&s, 0, sizeof s);
  s.c = c;
  s.t = &c->terms[un[0]];
  s.kind = un[1];
  s.f[0] = un[2];
  s.f[1] = un[3];
  for (int level = 1; level <= k - 2; ++level) {
    const int p = level + 1;
    for (int b = 0; b < s.t->nb[p]; ++b)
      __atomic_fetch_add(&c->levcnt[(int64_t)s.f[s.t->bq[p][b]] * (k - 2) + (level - 1)], 1, __ATOMIC_RELAXED);
    if (level == k - 2) break; /* the next node is a leaf: it accesses nothing */
    const int64_t nv = ivm_candidates(&s, p, cand);
    if (nv == 0) break;
    s.f[p] = cand[opcg_below(&r, (uint64_t)nv)];
    if (opcg_below(&r, (uint64_t)c->D) >= (uint64_t)nv) break; /* continue with probability |V|/D */
  }
}

typedef struct {
  pool_t *pool;
  const ivm_ctx *c;
} ow_arg;

static void *ow_worker(void *vp) {
  ow_arg *a = (ow_arg *)vp;
  int32_t *cand = (int32_t *)malloc(sizeof(int32_t) * (size_t)(a->c->D + 1));
  for (int64_t ch; (ch = pool_take(a->pool)) >= 0;)
    for (int64_t w = ch * 256; w < a->c->M && w < (ch + 1) * 256; ++w) ow_walk(a->c, w, cand);
  free(cand);
  return NULL;
}

typedef struct {
  pool_t *pool;
  const ivm_ctx *c;
  u128 added, removed;
} ivm_arg;

static void *ivm_worker(void *vp) {
  ivm_arg *a = (ivm_arg *)vp;
  const ivm_ctx *c = a->c;
  for (int64_t u; (u = pool_take(a->pool)) >= 0;) {
    const int32_t *un = c->units + 4 * u;
    ivm_state s;
    memset(&s, 0, sizeof s);
    s.c = c;
    s.t = &c->terms[un[0]];
    s.kind = un[1];
    s.f[0] = un[2];
    s.f[1] = un[3];
    ivm_visit(&s, 1);
    if (un[1] == 0) a->added += s.count;
    else a->removed += s.count;
  }
  return NULL;
}

/*
 * Enumerate the level-1 units (term, kind, a, b): every term i, every changed
 * edge of I (kind 0, "+") or D (kind 1, "-"), both orientations,
 * kept if L(a) = L_Q(u_x) and L(b) = L_Q(u_y). Returns the count;
 * writes up to cap units.
 */
int64_t ivm_units(int32_t k, int32_t m, const int32_t *qe, const int32_t *ql, const int32_t *user_order,
                  const int32_t *lab, int64_t n_ins, const int32_t *ins, int64_t n_del, const int32_t *del,
                  int32_t *units, int64_t cap) {
  oquery q;
  if (query_init(&q, k, m, qe, ql)) return -1;
  int uo[OMAXK], num[OMAXM][2], eidx[OMAXM];
  for (int i = 0; i < k; ++i) uo[i] = user_order ? user_order[i] : i;
  number_edges(&q, uo, eidx, num);
  int64_t nu = 0;
  for (int i = 0; i < m; ++i)
    for (int kind = 0; kind < 2; ++kind) {
      const int64_t ne = kind ? n_del : n_ins;
      const int32_t *E = kind ? del : ins;
      for (int64_t e = 0; e < ne; ++e)
        for (int o = 0; o < 2; ++o) {
          const int32_t a = o ? E[2 * e + 1] : E[2 * e], b = o ? E[2 * e] : E[2 * e + 1];
          if (!label_ok(lab, &q, num[i][0], a) || !label_ok(lab, &q, num[i][1], b)) continue;
          if (nu < cap) {
            units[4 * nu] = i; units[4 * nu + 1] = kind; units[4 * nu + 2] = a; units[4 * nu + 3] = b;
          }
          nu++;
        }
    }
  return nu;
}

/*
 * Run the IVM nested loops over the given units on the three views
 * (STABLE = E∩E', OLD = E, NEW = E'), each a CSR over the same n.
 * mode 0: out_counts[0..3] = added lo/hi, removed lo/hi.
 * mode 1: access[n] += number of tree nodes (levels 1..k-2) reading v's list.
 * mode 2: M plain random walks (ow_walk, seeded by `seed`); levcnt[n*(k-2)] += number of walks whose level-l
 *         node (1..k-2) reads v's list; N1 = n_units, D.
 */
int ivm_run(int32_t mode, int32_t n, const int64_t *rp_s, const int32_t *col_s, const int64_t *rp_o,
            const int32_t *col_o, const int64_t *rp_n, const int32_t *col_n, const int32_t *lab, int32_t k, int32_t m,
            const int32_t *qe, const int32_t *ql, const int32_t *user_order, int64_t n_units, const int32_t *units,
            int32_t threads, uint64_t seed, int64_t M, int64_t D, uint64_t *out_counts,
            uint64_t *access, uint64_t *levcnt) {
  oquery q;
  if (query_init(&q, k, m, qe, ql)) return -1;
  ograph gs = {n, rp_s, col_s}, go = {n, rp_o, col_o}, gn = {n, rp_n, col_n};
  ivm_ctx *c = (ivm_ctx *)calloc(1, sizeof(ivm_ctx));
  c->g[V_STABLE] = &gs; c->g[V_OLD] = &go; c->g[V_NEW] = &gn;
  c->lab = lab; c->q = &q; c->mode = mode;
  c->seed = seed; c->M = M; c->N1 = n_units; c->D = D;
  c->access = access; c->levcnt = levcnt; c->n_units = n_units; c->units = units;
  int uo[OMAXK], num[OMAXM][2], eidx[OMAXM];
  for (int i = 0; i < k; ++i) uo[i] = user_order ? user_order[i] : i;
  number_edges(&q, uo, eidx, num);
  for (int i = 0; i < m; ++i) build_term(&q, uo, num, i, &c->terms[i]);
  if (c->D < 1) { /* D must bound every list length (reading R19) */
    int64_t d = 1;
    for (int v = 0; v < n; ++v) {
      if (rp_o[v + 1] - rp_o[v] > d) d = rp_o[v + 1] - rp_o[v];
      if (rp_n[v + 1] - rp_n[v] > d) d = rp_n[v + 1] - rp_n[v];
    }
    c->D = d;
  }
  if (threads < 1) threads = 1;
  void *ptrs[256];
  if (mode == 2) {
    pool_t wpool = {(M + 255) / 256, 0, PTHREAD_MUTEX_INITIALIZER, NULL};
    ow_arg wargs[256];
    if (n_units > 0 && k > 2)
      for (int t = 0; t < threads && t < 256; ++t) { wargs[t] = (ow_arg){&wpool, c}; ptrs[t] = &wargs[t]; }
    if (n_units > 0 && k > 2) run_threads(threads, ow_worker, ptrs);
    free(c);
    return 0;
  }
  pool_t pool = {n_units, 0, PTHREAD_MUTEX_INITIALIZER, NULL};
  ivm_arg *args = (ivm_arg *)calloc((size_t)threads, sizeof(ivm_arg));
  for (int t = 0; t < threads && t < 256; ++t) { args[t] = (ivm_arg){&pool, c, 0, 0}; ptrs[t] = &args[t]; }
  run_threads(threads, ivm_worker, ptrs);
  u128 ad = 0, rm = 0;
  for (int t = 0; t < threads && t < 256; ++t) { ad += args[t].added; rm += args[t].removed; }
  if (out_counts) {
    out_counts[0] = (uint64_t)ad; out_counts[1] = (uint64_t)(ad >> 64);
    out_counts[2] = (uint64_t)rm; out_counts[3] = (uint64_t)(rm >> 64);
  }
  free(args);
  free(c);
  return 0;
}
