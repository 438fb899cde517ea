/*
 * gcsm.h — C ABI of the B200-native GCSM incremental-matching hot path.
 *
 * Paper: "GCSM: GPU-Accelerated Continuous Subgraph Matching for Large
 * Graphs" (Wei & Jiang, IPDPS). Citations "P:<line>" point into PAPER.md;
 * "R<n>" are the readings listed in DESIGN.md §3 (where the paper is silent or
 * garbled). Plain C types only: host pointers unless stated, sizes in
 * elements, no ownership transfer (every input is caller-owned and only read
 * during the call; every output is caller-allocated).
 *
 * Problem: a vertex-labelled undirected simple data graph
 * G_t = (V, E_t, L) on the fixed id universe [0, n) (R9) receives batches of
 * edge insertions I and deletions D; G_{t+1} = (E_t \ D) ∪ I (R8). For a
 * connected query Q (2 <= k <= 8 vertices, R10) the library returns
 *   added   = |Emb(Q, G_{t+1}) \ Emb(Q, G_t)|,
 *   removed = |Emb(Q, G_t) \ Emb(Q, G_{t+1})|,
 * where Emb is the set of injective, label- and edge-preserving maps
 * V(Q) -> V(G) (non-induced, R1-R3). Subgraph counts are embeddings divided
 * by gcsm_query_automorphisms().
 *
 * Pipeline of one gcsm_apply_batch (Fig. 3):
 *   (1) append / mark the batch on the host store
 *   (2) random-walk access-frequency estimation          P:183-260, eq. (3)
 *   (3) pack the top vertices' lists, one DMA to HBM
 *   (4) incremental matching on the GPU (eq. (1) terms)
 *       cached lists from HBM, the rest zero-copy from the pinned host store
 *   (4b) world > 1: one NCCL allreduce of the counters  (BASELINE north_star)
 *   (5) reorganise the updated host lists (merge)
 *
 * Status conventions:
 *   GCSM_EINVAL  bad argument, detected before any mutation (state unchanged);
 *   GCSM_ENOMEM  host / device allocation failure;
 *   GCSM_EDEVICE CUDA error: the context is poisoned;
 *   GCSM_ENCCL   NCCL error: the context is poisoned;
 *   GCSM_ESTATE  poisoned context, or apply_batch before set_query;
 *   GCSM_ETRUNC  list mode only: a tuple buffer was too small; the counts are
 *                still exact and the batch has been applied.
 * Threading: one context per host thread. With world > 1 the calls
 * set_query, set_cache_budget and apply_batch* are collective (every rank
 * calls them in the same order with identical arguments, like NCCL).
 */
#ifndef GCSM_H_
#define GCSM_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct gcsm_ctx gcsm_ctx; /* opaque, library-owned */

typedef enum {
  GCSM_OK = 0,
  GCSM_EINVAL = 1,
  GCSM_ENOMEM = 2,
  GCSM_EDEVICE = 3,
  GCSM_ENCCL = 4,
  GCSM_ESTATE = 5,
  GCSM_ETRUNC = 6
} gcsm_status;

/* Cache policies (step 3). ESTIMATOR is the paper's; the others are
 * the paper's comparison points run on the same kernels. */
enum {
  GCSM_CACHE_ESTIMATOR = 0, /* random-walk estimates, highest first */
  GCSM_CACHE_DEGREE = 1,    /* "Naive": degree as the frequency estimate */
  GCSM_CACHE_NONE = 2       /* "ZP": pure zero-copy regardless of the budget */
};

/* Option flags */
enum {
  GCSM_FLAG_LOCAL_COUNTS = 1u, /* world > 1 without NCCL: return this rank's shard counts
                                  (single-GPU "emulated world" used by the parity tests) */
  GCSM_FLAG_NO_SYMMETRY = 2u   /* count mode walks every embedding instead of one per Aut_L(Q) orbit
                                  (symmetry breaking is on by default; list mode never uses it) */
};

typedef struct {
  int32_t device;          /* CUDA ordinal; -1 = the current device */
  int32_t rank, world;     /* world = 1: single GPU */
  const void *nccl_id;     /* 128-byte ncclUniqueId (gcsm_nccl_unique_id on rank 0, broadcast by the
                              caller, e.g. through torch.distributed): required when world > 1, optional
                              with world = 1 (a one-rank communicator); NULL with GCSM_FLAG_LOCAL_COUNTS */
  uint64_t seed;           /* estimator RNG seed (R22) */
  int32_t host_threads;    /* 0 = all cores */
  int32_t cache_policy;    /* GCSM_CACHE_* */
  uint64_t walks_override; /* 0 = M = |ΔE| D^(k-2) / 32^k (R21) */
  uint32_t flags;          /* GCSM_FLAG_* */
  uint32_t reserved;
  int64_t vertex_capacity; /* ids the graph may grow into: 0 = n (no growth). Insertions may name ids in
                              [n, vertex_capacity): new vertices, each given an empty list with the average
                              degree as capacity; gcsm_add_vertices adds labelled ones */
  uint64_t staging_bytes;  /* per-GPU HBM for the fetch-once staging of zero-copy lists within a batch (DESIGN.md
                              §1d; two arenas, one per in-flight batch; not a cache: emptied every batch):
                              0 = default (a quarter of the free HBM when first needed, at most 32 GiB), 1 = off */
  int32_t store_rank, store_world; /* node-shared host store ("one shared shm arena cudaHostRegister'ed
                              in each process"). store_world = 1 (default): this context owns a private
                              pinned store. store_world = R in [2, 16]: the R local processes (one GPU each) share ONE
                              pinned, GPU-mapped store: store_rank 0 creates it from row_ptr / col / labels and returns
                              its handle from gcsm_store_handle(); ranks 1..R-1 pass that handle in store_handle
                              (row_ptr / col / labels are then ignored and may be NULL; n must match) after rank 0's
                              gcsm_create returned. The batch calls become collective over the R ranks (identical
                              batches, same order): each rank writes the overlays and merges of the updated vertices
                              it owns (x % R == store_rank) behind process-shared barriers. No id growth
                              (vertex_capacity must be 0 or n). A rank that fails a batch poisons the others' next
                              barrier (ESTATE); a barrier waits at most GCSM_SHM_TIMEOUT seconds (default 600). */
  const char *store_handle; /* NULL on store_rank 0; the creating rank's gcsm_store_handle() string elsewhere */
} gcsm_options;

/* Per-batch statistics (Table II-style breakdown; hit rate §8d). */
typedef struct {
  uint64_t batches;         /* batches applied so far */
  uint64_t n_ins, n_del;    /* normalised insertions / deletions of the last batch */
  uint64_t dropped;         /* no-op updates dropped by normalisation (R8) */
  uint64_t units;           /* level-1 units (term, oriented seed) processed on this rank */
  uint64_t n1;              /* |ΔE| of eq. (3): units of this rank (R15) */
  uint64_t walks;           /* M */
  uint64_t max_degree;      /* D (R19) */
  uint64_t cached_vertices; /* K */
  uint64_t cache_bytes;     /* bytes of cached lists (<= budget) */
  uint64_t hit_bytes;       /* list bytes the kernels read from the HBM cache (algorithmic, §8d) */
  uint64_t miss_bytes;      /* list bytes the kernels read zero-copy from host memory */
  uint64_t delta_bytes;     /* list bytes read from device-resident batch data: the ins/del segments of updated
                               vertices and (GPU estimator path) their stable lists S(x), uploaded with the batch */
  uint64_t hit_bytes_ext, miss_bytes_ext, delta_bytes_ext; /* the same, k_extend only (levels >= 3) */
  uint64_t host_copied_bytes; /* bytes the kernels bulk-copied from host memory (staging; real zero-copy reads) */
  uint64_t frontier;        /* level-2 partial matches materialised */
  uint64_t kernel_launches; /* this library's kernels launched in the last batch */
  uint64_t h2d_bytes;       /* bytes copied host -> device in the batch (cache DMA, descriptors, deltas, units) */
  uint64_t d2h_bytes;       /* bytes copied device -> host (counters, tuples) */
  uint64_t added, removed;  /* last batch's global counts */
  double ms_normalize;      /* (1) normalise + overlay + units */
  double ms_estimate;       /* (2) host part: level-1 walk roots on the GPU path (default), all walks with
                               GCSM_HOST_EST=1 */
  double ms_pack;           /* (3) host part: descriptors / staging (GPU path), ranking + layout (host path) */
  double ms_copy;           /* (3) GPU path: uploads + walks + ranking + cache copy on the stream (CUDA events);
                               host path: H2D of the cache, descriptors and deltas */
  double ms_match;          /* (4) kernels (CUDA events) */
  double ms_level2;         /* (4) k_level2 launches only (CUDA events) */
  double ms_extend;         /* (4) k_extend launches only (CUDA events) */
  double ms_allreduce;      /* (4b) */
  double ms_merge;          /* (5) */
  double ms_total;          /* whole gcsm_apply_batch, host wall clock */
  uint64_t stage_fill_bytes; /* bytes copied host -> the batch's staging arena (fetch-once staging; each list at
                                most once per batch; included in host_copied_bytes) */
  uint64_t stage_lists;      /* lists staged */
  uint64_t stage_hit_bytes;  /* algorithmic list bytes then served from the arena (HBM) instead of zero-copy */
  uint64_t bcomp_hit_bytes, bcomp_miss_bytes, bcomp_delta_bytes; /* B_comp: bytes of the DISTINCT
                                main lists the query's kernels touched, by home (HBM cache / pinned host / uploaded
                                lists of U); only with GCSM_BCOMP=1 at create (measurement mode), else 0 */
  uint64_t peer_bytes;       /* algorithmic list bytes read from a linked peer's HBM cache (gcsm_link_peers) */
  uint64_t walk_fill_bytes;  /* bytes the GPU walks (step 2) fetched into the staging arena (all queries) */
  uint64_t walk_stage_lists; /* lists they staged */
  uint64_t walk_alg_bytes;   /* this query's walks: algorithmic list bytes (driver scans + probed lists, §8d) */
  double ms_walks;           /* this query's GPU walk kernels (k_walks_l1 + k_walks, CUDA events; 0 if none) */
} gcsm_stats;

/* Fills *opt with the defaults (device -1, world 1, seed 0x6C53, all cores,
 * estimator cache policy, M from P:339). */
void gcsm_default_options(gcsm_options *opt);

/* Creates a context from the symmetric CSR of G_0: row_ptr[n+1]
 * (int64, because adjacency can exceed 2^31 entries), col[row_ptr[n]]; every
 * row sorted ascending, no duplicates, no self loops, symmetric, ids in
 * [0, n). labels: n values in [0, 65535], or NULL (unlabelled, R5).
 * The graph is copied into the library's pinned, GPU-mapped host store with
 * 2x capacity per list. opt may be NULL (defaults). EINVAL on any
 * violation (nothing allocated). With world > 1 and an nccl_id the NCCL
 * communicator is created by the first batch call (collective), so that a
 * node-shared store's rank 0 can return from gcsm_create and hand its store
 * handle to the other ranks first. Per-vertex device arrays are sized for
 * opt->vertex_capacity ids. */
gcsm_status gcsm_create(int32_t n, const int64_t *row_ptr, const int32_t *col, const int32_t *labels,
                        const gcsm_options *opt, gcsm_ctx **out);

/* Cross-process NVLink peer cache over a node-shared store: collective over the
 * store's ranks, after gcsm_set_cache_budget and with no batch in flight. Every rank exports its two cache
 * buffers, its two per-batch descriptor arrays and two interprocess events (CUDA IPC handles in its mailbox of the
 * shared mapping) and opens every other rank's (peer access enabled lazily). From the next batch on, a list
 * missing from this rank's cache is looked up in the peers' caches of the same batch (their descriptor array, one
 * 16-byte read over NVLink per peer) before the staging arena and zero-copy; each batch adds one store barrier
 * (every rank's cache step of batch t is enqueued), after which the matching waits (device) for the peers' cache
 * steps. The cache buffers are then fixed: gcsm_set_cache_budget may lower the budget but a larger one is EINVAL.
 * EINVAL without a shared store or with more than 7 peers; ESTATE before the
 * budget, with a batch in flight or when already linked; EDEVICE if a handle cannot be opened (the store's other
 * ranks then fail at their next barrier). */
gcsm_status gcsm_link_store_peers(gcsm_ctx *ctx);

/* Handle of a node-shared store (gcsm_options.store_world > 1) created by this context (store_rank 0): a
 * NUL-terminated path (the creating process's memfd under /proc) written to buf[cap]. The other local ranks
 * pass it as gcsm_options.store_handle while this process is alive. EINVAL for a private store or a buffer
 * shorter than the handle. */
gcsm_status gcsm_store_handle(const gcsm_ctx *ctx, char *buf, uint64_t cap);

/* Sets the query pattern: k vertices (2..8), m edges qedges[2m] over [0,k)
 * (undirected, simple, connected), qlabels[k] or NULL (any label), and the
 * user matching order order[k] (a permutation of [0,k)) or NULL (identity).
 * Builds the m IVM terms of eq. (1) as in Fig. 2b-f with the
 * stable-split views (R7, R11, R12). EINVAL leaves the previous query. */
gcsm_status gcsm_set_query(gcsm_ctx *ctx, int32_t k, int32_t m, const int32_t *qedges, const int32_t *qlabels,
                           const int32_t *order);

/* Adds another standing query to the context (gcsm_set_query replaces all of them with one). Arguments as
 * gcsm_set_query; *qid (may be NULL) receives its index (query 0 is the set_query one). Up to 32 queries. The
 * queries share the host store, each batch's normalisation, overlays and merge (steps (1) and (5) of Fig. 3)
 * and ONE device cache under the per-GPU budget, filled by ranking vertices on the SUM of the queries'
 * estimated access frequencies (eq. (3) per query; P:339's top-K rule on the sum). Every query gets
 * its own level-1 units, estimator walks, kernels and counters: gcsm_apply_batch / gcsm_wait_batch return
 * query 0's counts, gcsm_get_query_stats any query's. List mode needs exactly one query (EINVAL otherwise).
 * ESTATE before gcsm_set_query or with a batch in flight; EINVAL for a bad pattern or a 9th query (nothing
 * changes). With world > 1 this is collective. */
gcsm_status gcsm_add_query(gcsm_ctx *ctx, int32_t k, int32_t m, const int32_t *qedges, const int32_t *qlabels,
                           const int32_t *order, int32_t *qid);

/* Number of standing queries (0 before gcsm_set_query). */
int32_t gcsm_num_queries(const gcsm_ctx *ctx);

/* Per-GPU byte budget of the HBM list cache ("GPU buffer"); it counts
 * cached list payload (16-byte aligned lists). 0 = pure zero-copy. Applies
 * from the next batch. ENOMEM if the device buffer cannot be allocated. */
gcsm_status gcsm_set_cache_budget(gcsm_ctx *ctx, uint64_t bytes);

/* Applies one batch: ins[2*n_ins], del[2*n_del] (pairs of vertex ids, any
 * orientation; duplicates collapse; inserting an existing edge or deleting an
 * absent one is a counted no-op, R8). An insertion may name ids in [n, vertex_capacity): those vertices join
 * the graph. EINVAL (no mutation) on a self loop, an id outside [0, vertex_capacity), a deletion
 * naming an id >= n (deletions involve existing vertices), or an edge in both lists. On success *added /
 * *removed are the global embedding counts (every rank gets the same values). */
gcsm_status gcsm_apply_batch(gcsm_ctx *ctx, int64_t n_ins, const int32_t *ins, int64_t n_del, const int32_t *del,
                             uint64_t *added, uint64_t *removed);

/* Like gcsm_apply_batch, also listing the changed embeddings as k-tuples in
 * query-vertex order (tuple[u] = f(u)): up to added_cap / removed_cap tuples
 * (k int32 each) into added_tuples / removed_tuples. Single-GPU (world == 1 or
 * GCSM_FLAG_LOCAL_COUNTS). Tuple order is unspecified. ETRUNC if a buffer was
 * too small (counts exact, batch applied). */
gcsm_status gcsm_apply_batch_list(gcsm_ctx *ctx, int64_t n_ins, const int32_t *ins, int64_t n_del, const int32_t *del,
                                  int32_t *added_tuples, uint64_t added_cap, int32_t *removed_tuples,
                                  uint64_t removed_cap, uint64_t *added, uint64_t *removed);

/* Pipelined form of gcsm_apply_batch (overlap batch t+1's host steps (1)-(3) with batch
 * t's kernels). gcsm_submit_batch validates and normalises the batch (EINVAL without mutation as above), runs
 * its host steps, enqueues its GPU work and its count allreduce on the library's stream, and merges it into
 * the host store (G_{t+1} is the store's state on return) without waiting for the kernels: the merge writes
 * fresh arrays, and the arrays an in-flight batch may read are recycled only after it completes (P:302's
 * consistency). At most two batches may be outstanding (ESTATE otherwise). gcsm_wait_batch waits for the
 * oldest outstanding batch and returns its counts (ESTATE if none); gcsm_get_stats then describes it.
 * gcsm_apply_batch(_list) = submit + wait (draining older submissions first). set_query and set_cache_budget
 * return ESTATE while a batch is outstanding. With world > 1 both calls are collective. */
gcsm_status gcsm_submit_batch(gcsm_ctx *ctx, int64_t n_ins, const int32_t *ins, int64_t n_del, const int32_t *del);
gcsm_status gcsm_wait_batch(gcsm_ctx *ctx, uint64_t *added, uint64_t *removed);

/* Last batch's statistics (query 0; the shared steps' times are the batch's). */
gcsm_status gcsm_get_stats(const gcsm_ctx *ctx, gcsm_stats *out);

/* Last batch's statistics of query qid (its counts in added / removed, its kernels' times and bytes, its
 * estimator time; the shared steps as in gcsm_get_stats). EINVAL for an unknown qid. */
gcsm_status gcsm_get_query_stats(const gcsm_ctx *ctx, int32_t qid, gcsm_stats *out);

/* |Aut_L(Q)| (label-preserving automorphisms) of the current query, 0 if none. */
uint64_t gcsm_query_automorphisms(const gcsm_ctx *ctx);

/* Static-lifetime (per ctx) message for the last error; "" if none. */
const char *gcsm_last_error(const gcsm_ctx *ctx);

/* Current number of vertices (ids [0, n)); grows by insertions naming new ids or gcsm_add_vertices. */
int32_t gcsm_num_vertices(const gcsm_ctx *ctx);

/* Adds `count` isolated vertices (ids n .. n+count-1, *first_id = n) with labels[count] (NULL: label 0), each
 * with an empty list of the average degree's capacity. EINVAL beyond the vertex capacity
 * (gcsm_options.vertex_capacity) or for labels on an unlabelled graph; ESTATE with a batch in flight. */
gcsm_status gcsm_add_vertices(gcsm_ctx *ctx, int32_t count, const int32_t *labels, int32_t *first_id);

/* NVLink peer cache (host data movement is the bottleneck): links n contexts
 * (2 <= n <= 8) of this process — one per GPU, or several on one GPU — so that a list missing from a context's
 * own HBM cache is read from a linked context's HBM cache (peer access over NVLink / NVSwitch) before falling
 * back to zero-copy host reads. The contexts must hold the same graph and apply the same batches in lockstep
 * (same vertex capacity and batch count at link time), each driven by ITS OWN host thread: a context's submit
 * of batch t waits (host rendezvous) until every linked context has enqueued its cache step of batch t, and its
 * matching kernels wait (device events) for those cache steps; a context's cache step of batch t+2 waits for
 * every peer's batch t. n = 0 or 1 unlinks the given contexts (gcsm_destroy also unlinks the group).
 * EINVAL on bad arguments or a mismatch, ESTATE with a batch in flight, EDEVICE without peer access. */
gcsm_status gcsm_link_peers(gcsm_ctx *const *ctxs, int32_t n);

/* Measurement modes for the following batches (flags = GCSM_MEASURE_*; 0 = off, the default). With
 * GCSM_MEASURE_BCOMP the kernels also mark, per query, the vertices whose main list they read, and the batch's
 * statistics report B_comp (bytes of the DISTINCT lists touched, by home: HBM cache, pinned host,
 * uploaded lists of U) in bcomp_*_bytes; it costs one atomic per list read and serialises each batch's
 * kernels on the context stream, so timed runs leave it off. EINVAL for unknown flags, ENOMEM if the bitmap
 * (n bits) cannot be allocated. Also enabled at create by the environment variable GCSM_BCOMP=1. */
enum { GCSM_MEASURE_BCOMP = 1u };
gcsm_status gcsm_set_measure(gcsm_ctx *ctx, uint32_t flags);

/* Frees everything (pinned store, device buffers, stream, communicator). NULL-safe. */
void gcsm_destroy(gcsm_ctx *ctx);

/* ---------------------------------------------------------------- evidence helpers */

/* 128-byte ncclUniqueId for rank 0 to broadcast (world > 1). */
gcsm_status gcsm_nccl_unique_id(void *out128);

/* CUDA stream (cudaStream_t) the library launches on, so a caller can time it. */
gcsm_status gcsm_get_stream(const gcsm_ctx *ctx, void **stream);

/* Current graph as symmetric CSR: row_ptr[n+1] always written; col written
 * if col_cap >= row_ptr[n], else ETRUNC. */
gcsm_status gcsm_export_csr(const gcsm_ctx *ctx, int64_t *row_ptr, int32_t *col, uint64_t col_cap);

/* Last batch's estimator output (step 2) for query 0: the vertices with a non-zero count,
 * ascending, and per vertex the per-level sums of walk multiplicities B for
 * tree levels 1..k-2 (eq. (3)): levcnt[i*8 + (l-1)]. *n_out = the number of
 * such vertices (ETRUNC if > cap; the first cap are written). On the GPU path the
 * sums live in device memory: the call synchronises the context's streams. */
gcsm_status gcsm_get_estimates(const gcsm_ctx *ctx, int32_t *ids, uint64_t *levcnt, uint64_t cap, uint64_t *n_out);

/* Last batch's cached vertex set (step 3), ascending: the longest prefix of (estimate desc, id asc)
 * that fits the budget (R23), over the vertices not updated by the batch on the GPU path (their
 * stable lists are uploaded with the batch, R32). Synchronises the context's streams. */
gcsm_status gcsm_get_cached(const gcsm_ctx *ctx, int32_t *ids, uint64_t cap, uint64_t *n_out);

/* Roofline denominators the hot path needs and MEASURED_PEAKS.json lacks
 * (SURVEY §8d): best-of-5 GB/s of (i) a zero-copy streaming-read kernel over a
 * mapped pinned buffer of `bytes`, (ii) one cudaMemcpyAsync H2D of it, and
 * (iii) an HBM device copy (read + write bytes). device -1 = current. */
gcsm_status gcsm_measure_host_link(int32_t device, uint64_t bytes, double *zero_copy_gbps, double *dma_h2d_gbps,
                                   double *hbm_copy_gbps);

/* Pure host, no device: the per-term plan the library would build for a query
 * (for the Fig. 2 structural test). Arrays as in gcsm_set_query; outputs:
 * out_seed[2m] (numbered query edges R_1..R_m), out_order[m*k],
 * out_nb[m*k] (backward edges per term position), out_bq[m*k*8] (backward
 * positions), out_view[2*m*k*8] (view per backward edge for + / - terms:
 * 0 stable, 1 old N, 2 new N'). */
gcsm_status gcsm_plan_inspect(int32_t k, int32_t m, const int32_t *qedges, const int32_t *order, int32_t *out_seed,
                              int32_t *out_order, int32_t *out_nb, int32_t *out_bq, int32_t *out_view);

/* Pure host, no device: the symmetry-breaking restrictions the library uses for a query in count mode
 * (Grochow-Kellis on Aut_L(Q), user order as the vertex order): pairs (u, w) meaning f(u) < f(w); exactly one
 * embedding per Aut_L orbit satisfies all of them. out_pairs[2*cap]; *n_out = the number of pairs (ETRUNC if
 * > cap); *aut = |Aut_L(Q)|. */
gcsm_status gcsm_query_restrictions(int32_t k, int32_t m, const int32_t *qedges, const int32_t *qlabels,
                                    const int32_t *order, int32_t *out_pairs, int32_t cap, int32_t *n_out,
                                    uint64_t *aut);

/* Pure host, no device: the estimator's binomial sampler (§IV-B: B ~ Bin(n, p)), as the walks draw it:
 * out[i] = Bin(n, p) drawn from the counter-based key chain(key0, i) (reading R22; BINV for n p < 10, BTRD
 * otherwise, R20). For the distribution tests of the product's sampler (chi-square against the exact pmf).
 * count >= 0, n >= 0, 0 <= p <= 1, else EINVAL. */
gcsm_status gcsm_binomial_samples(uint64_t key0, int64_t n, double p, int64_t count, int64_t *out);

/* Pure host, no device: the shard of each unit for world ranks (LPT on the
 * cost proxy cost[i], ties by index): out_rank[n_units]. */
gcsm_status gcsm_shard(int64_t n_units, const uint64_t *cost, int32_t world, int32_t *out_rank);

#ifdef __cplusplus
}
#endif
#endif /* GCSM_H_ */
