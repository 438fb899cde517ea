// gcsm.cpp — the C ABI (include/gcsm.h) and the per-batch pipeline (Fig. 3).
#include "gcsm.h"

#include <cuda_runtime.h>
#include <nccl.h>

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <condition_variable>
#include <cstring>
#include <memory>
#include <mutex>
#include <new>
#include <numeric>
#include <string>
#include <vector>

#include "estimator.h"
#include "internal.h"
#include "estimator_gpu.cuh"
#include "kernels.cuh"
#include "stage.cuh"
#include "store.h"

using namespace gcsm;

namespace {

constexpr int64_t kF2CapLimit = 64ll << 20;  // level-2 frontier entries per chunk

// Growth inside a submit must not wait for the previous batch's kernels: device buffers are re-allocated
// stream-ordered on the context's stream (cudaFreeAsync / cudaMallocAsync), replaced pinned buffers are parked
// until the context is destroyed (cudaFreeHost would synchronise the device). Set by submit_impl.
thread_local cudaStream_t g_alloc_stream = nullptr;
thread_local std::vector<void *> *g_retired_pinned = nullptr;

template <typename T>
bool dev_ensure(T *&p, size_t &cap, size_t need) {
  if (need <= cap && p) return true;
  if (p) {
    if (g_alloc_stream) cudaFreeAsync(p, g_alloc_stream);
    else cudaFree(p);
  }
  p = nullptr;
  cap = 0;
  size_t n = std::max<size_t>(need, 1);
  n = 2 * n;
  if (g_alloc_stream) {
    if (cudaMallocAsync((void **)&p, n * sizeof(T), g_alloc_stream) != cudaSuccess) return false;
  } else if (cudaMalloc((void **)&p, n * sizeof(T)) != cudaSuccess) {
    return false;
  }
  cap = n;
  return true;
}

template <typename T>
bool host_ensure(T *&p, size_t &cap, size_t need) {
  if (need <= cap && p) return true;
  if (p) {
    if (g_retired_pinned) g_retired_pinned->push_back(p);
    else cudaFreeHost(p);
  }
  p = nullptr;
  cap = 0;
  size_t n = std::max<size_t>(need, 1);
  n = 2 * n;
  if (cudaHostAlloc((void **)&p, n * sizeof(T), cudaHostAllocDefault) != cudaSuccess) return false;
  cap = n;
  return true;
}

// NVLink peer cache: contexts linked by gcsm_link_peers read each other's HBM caches. The
// per-batch rendezvous below orders the cross-context reads: a context's matching of batch t starts
// after every peer's cache step of batch t (their descriptors and cache are final), and a context's cache step of
// batch t+2 (which rewrites the slot and buffer of batch t) waits for every peer's batch t.
struct PeerGroup {
  std::mutex mu;
  std::condition_variable cv;
  std::vector<gcsm_ctx *> members;
  std::vector<uint64_t> enq;  // per member: batches whose cache step has been enqueued
};

// Cross-process peer cache over a node-shared store (gcsm_link_store_peers): what each rank publishes in its
// mailbox of the shared mapping, and what it opened of the others'.
struct PeerMail {
  cudaIpcMemHandle_t cache[2], vdesc[2];
  cudaIpcEventHandle_t ev[2];
  uint64_t cache_va[2];
  uint64_t cache_cap;
  int32_t device, linked;
  volatile int32_t cache_idx[2];  // per slot: the cache buffer (0 / 1) batch t's kernels read, -1 none
};
static_assert(sizeof(PeerMail) <= kShmMailBytes, "mailbox");
struct StorePeers {
  int n = 0;
  int rank[GCSM_MAX_PEERS] = {};
  void *vdesc[GCSM_MAX_PEERS][2] = {};
  char *cache_map[GCSM_MAX_PEERS][2] = {};
  uint64_t cache_va[GCSM_MAX_PEERS][2] = {};
  uint64_t cache_cap[GCSM_MAX_PEERS] = {};
  cudaEvent_t ev[GCSM_MAX_PEERS][2] = {};
};

}  // namespace

struct gcsm_ctx {
  gcsm_options opt{};
  int device = 0;
  std::string err;
  bool poisoned = false;
  HostStore store;
  // Standing queries (gcsm_set_query sets query 0, gcsm_add_query appends): they share the host store, the batch
  // normalisation / overlays / merge and ONE cache under the per-GPU budget (ranked by the sum of the queries'
  // estimates); each has its own units, estimator run, plans, kernels and counters.
  struct Query {
    QueryPlan qp;   // plans without restrictions
    QueryPlan qps;  // plans with the symmetry-breaking restrictions of Aut_L(Q)
    DevPlan *d_plans = nullptr, *d_splans = nullptr;
    EstimatorOutput est;  // last batch's estimator output
    gcsm_stats stats{};   // last completed batch
  };
  std::vector<Query> qs;
  bool has_query = false;
  uint64_t budget = 0;
  cudaStream_t stream = nullptr;
  // Per in-flight batch state (double buffered: batch t's async copies read its pinned staging while batch
  // t+1's host steps fill the other slot; pipelined submit/wait).
  struct Slot {
    int64_t *h_pidx = nullptr; size_t h_pidx_cap = 0;
    VDesc *h_pval = nullptr; size_t h_pval_cap = 0;
    DRec *h_drec = nullptr; size_t h_drec_cap = 0;
    int32_t *h_dlist = nullptr; size_t h_dlist_cap = 0;
    Unit *h_units = nullptr; size_t h_units_cap = 0;
    uint64_t *h_gather = nullptr; size_t h_gather_cap = 0;
    uint64_t *h_fresh = nullptr; size_t h_fresh_cap = 0;
    unsigned long long *h_cnt = nullptr;  // CNT_N per query
    EstUnit *h_eunits = nullptr; size_t h_eunits_cap = 0;  // level-1 walk nodes (GPU estimator)
    int2 *h_eitems = nullptr; size_t h_eitems_cap = 0;     // their work items
    int32_t *h_ulist = nullptr; size_t h_ulist_cap = 0;    // stable lists S(x) of U, packed (GPU path)
    int4 *h_srec = nullptr; size_t h_srec_cap = 0;         // sampled-index updates of the previous batch's U
    int32_t *h_sstage = nullptr; size_t h_sstage_cap = 0;
    int32_t *d_ulist = nullptr; size_t d_ulist_cap = 0;    // their device copy (read by this batch's kernels)
    // per-batch device state (double buffered so that batch t+1's cache step can run while batch t matches):
    // descriptors (copied from the previous batch's, then patched), delta records and lists, units, counters
    VDesc *d_vdesc = nullptr;
    DRec *d_drec = nullptr; size_t drec_cap = 0;
    int32_t *d_dlist = nullptr; size_t dlist_cap = 0;
    Unit *d_units = nullptr; size_t units_cap = 0;
    int2 *d_useg = nullptr; size_t useg_cap = 0;
    unsigned long long *d_cnt = nullptr;  // CNT_N per query
    size_t ulist_n = 0;
    double *h_r0 = nullptr; size_t h_r0_cap = 0;           // BINV table staging
    cudaEvent_t ev_a0 = nullptr, ev_a1 = nullptr, ev_c0 = nullptr, ev_c1 = nullptr, ev_done = nullptr;
    cudaEvent_t ev_up = nullptr, ev_l2 = nullptr;  // uploads done (fork) / hoisted level-2 work done (join)
    struct PerQuery {
      cudaEvent_t ev_m0 = nullptr, ev_m1 = nullptr;
      std::vector<cudaEvent_t> kev;  // per frontier chunk: level2 start, extend start, extend end
      size_t nev = 0;
      uint64_t aut_mul = 1;  // canonical-embedding counts x |Aut_L| (symmetry breaking)
      gcsm_stats st{};
    };
    std::vector<PerQuery> q;
    bool inflight = false;
    double host_ms = 0;
    // list mode
    int32_t *tup_add = nullptr, *tup_rem = nullptr, *d_tadd = nullptr, *d_trem = nullptr;
    uint64_t add_cap = 0, rem_cap = 0;
    std::vector<std::pair<int32_t *, uint32_t>> retired;  // host arrays replaced by this batch's merge
    const char *cache_lo = nullptr, *cache_hi = nullptr;  // the HBM cache this batch's kernels read (peers too)
    std::vector<cudaEvent_t> ev_walk;  // 2 per query around its walk kernels
    bool walks_timed = false;
  };
  Slot slots[2];
  uint64_t waited = 0;  // batches whose results have been collected
  ncclComm_t comm = nullptr;
  bool comm_pending = false;       // the communicator is created at the first batch (collective)
  unsigned char nccl_id[128] = {};
  int grid = 0, warps_total = 0;
  int ext_grid = 0;  // blocks of the extension kernels (GCSM_EXT_RESERVE blocks left for the overlapped cache step)

  // device buffers
  uint16_t *d_lab = nullptr;
  int32_t *d_f2q[GCSM_MAX_QUERIES] = {};  size_t f2q_cap[GCSM_MAX_QUERIES] = {};  // per query: 2 * f2 entries ints
  int32_t *d_groupq[GCSM_MAX_QUERIES] = {};  size_t groupq_cap[GCSM_MAX_QUERIES] = {};  // frontier grouped by x2
  cudaStream_t stream2 = nullptr;  // GPU path: the first level-2 kernels run here, beside the cache step
  // GPU path: batch t+1's cache step (uploads, walks, ranking, k_copy, descriptor switch into its own descriptor
  // copy) runs here while batch t's extension kernels run on `stream` (GCSM_NO_OVERLAP=1 at create: on `stream`)
  cudaStream_t stream3 = nullptr;
  bool overlap = false;
  int overlap_kmax = 8;  // largest query size whose batches overlap the cache step (GCSM_OVERLAP_KMAX; C4 A/B:
                         // 100.4-100.8 ms per step with the overlap, 101.3-103.0 without, profiles/ab10_r02.txt)
  uint32_t *d_hist = nullptr;                         // n counters + scan
  uint32_t *d_bsum = nullptr;
  int32_t *d_scratch = nullptr; size_t scratch_cap = 0;
  char *d_cache = nullptr; size_t cache_cap = 0;   // the buffer this batch's kernels read
  char *d_cachebuf[2] = {nullptr, nullptr};        // double buffer: last batch's cache stays readable
  int cache_cur = 0;                               // buffer holding the previous batch's cache
  bool cache_valid = false;                        // slot16 describes d_cachebuf[cache_cur]
  std::vector<uint32_t> slot16;  // per vertex: 1 + (offset / 16) of its list in the previous cache, 0 = not cached
  uint64_t *d_gather = nullptr; size_t gather_cap = 0;  // retained lists: (src, dst, n16) triples
  uint64_t *d_fresh = nullptr; size_t fresh_cap = 0;    // newly cached lists: (host src, dst, n16) triples
  std::vector<int32_t> sel_index;                       // vertex -> index in this batch's selection, or -1
  int64_t *d_pidx = nullptr; size_t pidx_cap = 0;
  VDesc *d_pval = nullptr; size_t pval_cap = 0;
  int32_t *d_tup = nullptr; size_t tup_cap = 0;
  unsigned long long *d_red = nullptr; size_t red_cap = 0;  // packed (added, removed) of every query: one allreduce
  int32_t *d_arena = nullptr; size_t arena_cap = 0;     // level-3 work sharing (k >= 5)
  Task *d_tasks = nullptr; size_t tasks_cap = 0;
  int32_t *d_task_ready = nullptr; size_t task_ready_cap = 0;
  int32_t task_gen = 0;
  // GPU estimator + cache packer (steps 2-3 on the device, estimator_gpu.cu; default). GCSM_HOST_EST=1 at create
  // selects the host walker and host packer instead (the paper's CPU placement, kept for A/B measurements).
  bool gpu_est = true;
  bool gpu_ready = false;          // the n-sized buffers below exist
  bool cache_reset = false;        // the last selection's descriptors must go back to host before the next batch
  unsigned long long *d_hptr = nullptr;  // host address of every vertex's main list
  uint32_t *d_touched = nullptr, *d_wcnt = nullptr, *d_woff = nullptr;
  int32_t *d_tids = nullptr, *d_prev_sel = nullptr;
  unsigned long long *d_bits = nullptr, *d_bytes = nullptr, *d_scan = nullptr, *d_off = nullptr;
  uint8_t *d_flag = nullptr;
  unsigned long long *d_selhist = nullptr, *d_ecursor = nullptr;
  SelState *d_sel = nullptr;
  void *d_cubtmp = nullptr; size_t cubtmp_bytes = 0;
  unsigned long long *d_levcnt[GCSM_MAX_QUERIES] = {};
  int lev_levels[GCSM_MAX_QUERIES];  // -1 until allocated (set in gcsm_create)
  EstUnit *d_eunits = nullptr; size_t eunits_cap = 0;
  int2 *d_eitems = nullptr; size_t eitems_cap = 0;
  EstNode2 *d_ef2 = nullptr; size_t ef2_cap = 0;
  double *d_r0 = nullptr; size_t r0_cap = 0;
  double *d_sfc = nullptr;         // BTRD Stirling table (10 doubles)
  // sampled index of the host lists (every 32nd element of each list of >= 64 elements): lets k_last4 fetch only
  // the symmetry-range slice of a zero-copy list. Per-vertex slots, relocated to an append area when a merged list
  // outgrows its slot (none left: the vertex is not indexed and its lists are fetched whole)
  int32_t *d_sidx = nullptr; uint32_t *d_soff = nullptr;
  size_t sidx_capacity = 0, sidx_next = 0;
  std::vector<uint32_t> soff_h, scap_h;
  int4 *d_srec = nullptr; size_t srec_cap = 0;
  int32_t *d_sstage = nullptr; size_t sstage_cap = 0;
  size_t r0_n = 0;                 // entries of the device table of (1 - pD)^n
  double r0_pD = -1.0;
  bool est_valid = false;          // the device holds a batch's estimator output (gcsm_get_estimates)
  // fetch-once staging of zero-copy lists within a batch (kernels.cu stage_resolve): per-vertex
  // state words, the arena (emptied every batch: a new epoch) and its bump counter
  // one arena per in-flight slot: batch t+1's walks (cache step, possibly on its own stream) stage into their slot
  // while batch t's matching reads the other
  struct StageSlot {
    unsigned long long *state = nullptr;
    int32_t *arena = nullptr;
    size_t cap = 0;  // ints
    unsigned long long *bump = nullptr;
  } stg[2];
  bool stage_failed = false;       // allocation failed once: stay off
  uint32_t stage_min = 1;          // shortest list (ints) routed through the arena (GCSM_STAGE_MIN)
  uint32_t walk_stage_epoch = 0;   // this batch's walks stage through the arena too (0 = no)
  int32_t stage_policy = 1;        // smem staging model for device-resident probe lists (GCSM_STAGE_POLICY)
  int32_t walk_lane = 1;           // GCSM_WALK_LANE=0: level k-3 walk nodes by the warp-wide DFS (A/B)
  int32_t walk_stage = 1;          // staging of skip-sampled walk drivers (GCSM_WALK_STAGE: 0 always, 1 expected >= 1, 2 never)
  // B_comp measurement mode (GCSM_BCOMP=1 at create): bitmap of the vertices whose main list a query's kernels read
  uint32_t *d_touched_bc = nullptr;
  bool bcomp = false;
  std::vector<void *> retired_pinned;  // pinned staging replaced by a larger one (freed at destroy)
  // shared store: host arrays retired by batch t's merge, recycled once EVERY rank has collected batch t (at the
  // first barrier of batch t+2: a rank submits t+2 only after waiting for t)
  std::vector<std::pair<uint64_t, std::vector<std::pair<int32_t *, uint32_t>>>> pending_retired;


  // cache / batch state
  std::vector<int32_t> prev_cached, prev_U;
  std::vector<uint8_t> mark;         // scratch (n)
  EstimatorScratch est_scratch;
  uint64_t batch_seq = 0;
  std::vector<int32_t> degree_order;  // GCSM_CACHE_DEGREE ranking

  std::shared_ptr<PeerGroup> peers;  // gcsm_link_peers
  StorePeers sp;                      // gcsm_link_store_peers (other processes of the node-shared store)
  cudaEvent_t ev_ipc[2] = {nullptr, nullptr};  // per slot: this batch's cache step is complete (interprocess)
  int peer_idx = -1;
  bool in_batch = false;  // between a successful normalise and the end of submit: failures poison the ctx
  gcsm_status fail(gcsm_status s, const std::string &m) {
    err = m;
    if (s == GCSM_EDEVICE || s == GCSM_ENCCL || (in_batch && s != GCSM_EINVAL)) poisoned = true;
    if (poisoned) store.poison_shared();  // the other ranks of a shared store stop at their next barrier
    return s;
  }
  gcsm_status cuda_fail(cudaError_t e, const char *where) {
    return fail(GCSM_EDEVICE, std::string(where) + ": " + cudaGetErrorString(e));
  }
  ~gcsm_ctx();
};

#define CK(call)                                     \
  do {                                               \
    cudaError_t e_ = (call);                         \
    if (e_ != cudaSuccess) return ctx->cuda_fail(e_, #call); \
  } while (0)

static void peer_leave(gcsm_ctx *ctx);

static void store_peers_close(gcsm_ctx *ctx) {
  StorePeers &sp = ctx->sp;
  for (int p = 0; p < sp.n; ++p)
    for (int j = 0; j < 2; ++j) {
      if (sp.vdesc[p][j]) cudaIpcCloseMemHandle(sp.vdesc[p][j]);
      if (sp.cache_map[p][j]) cudaIpcCloseMemHandle(sp.cache_map[p][j]);
      if (sp.ev[p][j]) cudaEventDestroy(sp.ev[p][j]);
    }
  sp = StorePeers();
}

gcsm_ctx::~gcsm_ctx() {
  peer_leave(this);
  if (stream) cudaStreamSynchronize(stream);
  if (comm) ncclCommDestroy(comm);
  for (Query &q : qs)
    for (DevPlan *p : {q.d_plans, q.d_splans})
      if (p) cudaFree(p);
  if (stream3) cudaStreamSynchronize(stream3);
  store_peers_close(this);  // after this context's kernels (they may read the peers' memory) have finished
  for (cudaEvent_t e : ev_ipc)
    if (e) cudaEventDestroy(e);
  void *dev[] = {d_lab, d_scratch, d_red, d_cachebuf[0],
                 d_cachebuf[1], d_gather, d_pidx, d_pval, d_tup, d_hist, d_bsum, d_fresh, d_arena, d_tasks, d_task_ready};
  for (int q = 0; q < GCSM_MAX_QUERIES; ++q) {
    if (d_f2q[q]) cudaFree(d_f2q[q]);
    if (d_groupq[q]) cudaFree(d_groupq[q]);
  }
  for (void *p : dev)
    if (p) cudaFree(p);
  void *dev2[] = {d_hptr, d_touched, d_wcnt, d_woff, d_tids, d_prev_sel, d_bits, d_bytes, d_scan, d_off, d_flag,
                  d_selhist, d_ecursor, d_sel, d_cubtmp, d_eunits, d_r0, d_eitems, d_ef2, d_sfc, d_sidx, d_soff,
                  d_srec, d_sstage, d_touched_bc, stg[0].state, stg[0].arena, stg[0].bump, stg[1].state,
                  stg[1].arena, stg[1].bump};
  for (void *p : dev2)
    if (p) cudaFree(p);
  for (unsigned long long *p : d_levcnt)
    if (p) cudaFree(p);
  for (void *p : retired_pinned) cudaFreeHost(p);
  for (Slot &sl : slots) {
    void *host[] = {sl.h_pidx, sl.h_pval, sl.h_drec, sl.h_dlist, sl.h_units, sl.h_gather, sl.h_fresh, sl.h_cnt,
                    sl.h_eunits, sl.h_ulist, sl.h_r0, sl.h_eitems, sl.h_srec, sl.h_sstage};
    if (sl.d_ulist) cudaFree(sl.d_ulist);
    for (void *p : {(void *)sl.d_vdesc, (void *)sl.d_drec, (void *)sl.d_dlist, (void *)sl.d_units, (void *)sl.d_useg,
                    (void *)sl.d_cnt})
      if (p) cudaFree(p);
    for (void *p : host)
      if (p) cudaFreeHost(p);
    for (cudaEvent_t e : {sl.ev_a0, sl.ev_a1, sl.ev_c0, sl.ev_c1, sl.ev_done, sl.ev_up, sl.ev_l2})
      if (e) cudaEventDestroy(e);
    for (cudaEvent_t e : sl.ev_walk) cudaEventDestroy(e);
    for (auto &pq : sl.q) {
      for (cudaEvent_t e : {pq.ev_m0, pq.ev_m1})
        if (e) cudaEventDestroy(e);
      for (cudaEvent_t e : pq.kev) cudaEventDestroy(e);
    }
  }
  if (stream2) cudaStreamSynchronize(stream2);
  if (stream) cudaStreamDestroy(stream);
  if (stream2) cudaStreamDestroy(stream2);
  if (stream3) cudaStreamDestroy(stream3);
}

// Leaves the peer group (the remaining members are unlinked too: a group is all or nothing).
static void peer_leave(gcsm_ctx *ctx) {
  if (!ctx || !ctx->peers) return;
  std::shared_ptr<PeerGroup> pg = ctx->peers;
  std::lock_guard<std::mutex> lk(pg->mu);
  for (gcsm_ctx *p : pg->members) {
    p->peers.reset();
    p->peer_idx = -1;
  }
  pg->members.clear();
}

extern "C" {

void gcsm_default_options(gcsm_options *o) {
  if (!o) return;
  std::memset(o, 0, sizeof *o);
  o->device = -1;
  o->rank = 0;
  o->world = 1;
  o->seed = 0x6C53;
  o->host_threads = 0;
  o->cache_policy = GCSM_CACHE_ESTIMATOR;
  o->store_world = 1;
}

gcsm_status gcsm_nccl_unique_id(void *out128) {
  if (!out128) return GCSM_EINVAL;
  ncclUniqueId id;
  if (ncclGetUniqueId(&id) != ncclSuccess) return GCSM_ENCCL;
  std::memcpy(out128, &id, sizeof id);
  return GCSM_OK;
}

gcsm_status gcsm_create(int32_t n, const int64_t *row_ptr, const int32_t *col, const int32_t *labels,
                        const gcsm_options *opt, gcsm_ctx **out) {
  if (!out) return GCSM_EINVAL;
  *out = nullptr;
  gcsm_options o;
  gcsm_default_options(&o);
  if (opt) o = *opt;
  if (o.world < 1 || o.rank < 0 || o.rank >= o.world) return GCSM_EINVAL;
  if (o.world > 1 && !o.nccl_id && !(o.flags & GCSM_FLAG_LOCAL_COUNTS)) return GCSM_EINVAL;
  if (o.cache_policy < 0 || o.cache_policy > 2) return GCSM_EINVAL;
  if (o.store_world < 1) o.store_world = 1;
  const bool shared = o.store_world > 1;
  if (shared && (o.store_world > GCSM_MAX_STORE_RANKS || o.store_rank < 0 || o.store_rank >= o.store_world ||
                 (o.store_rank > 0) != (o.store_handle != nullptr) || (o.vertex_capacity != 0 && o.vertex_capacity != n)))
    return GCSM_EINVAL;
  if (n < 1 || (!row_ptr && !(shared && o.store_rank > 0))) return GCSM_EINVAL;
  gcsm_ctx *ctx = new (std::nothrow) gcsm_ctx();
  if (!ctx) return GCSM_ENOMEM;
  ctx->opt = o;
  int threads = o.host_threads > 0 ? o.host_threads : (int)std::max(1u, std::thread::hardware_concurrency());
  ctx->opt.host_threads = threads;
  // device
  int dev = o.device;
  if (dev < 0 && cudaGetDevice(&dev) != cudaSuccess) {
    delete ctx;
    return GCSM_EDEVICE;
  }
  if (cudaSetDevice(dev) != cudaSuccess) {
    delete ctx;
    return GCSM_EDEVICE;
  }
  ctx->device = dev;
  bool cuda_err = false;
  if (o.vertex_capacity < 0 || o.vertex_capacity > INT32_MAX) {
    delete ctx;
    return GCSM_EINVAL;
  }
  const int32_t ncap = (int32_t)std::max<int64_t>(n, o.vertex_capacity);
  std::string e = !shared ? ctx->store.init(n, row_ptr, col, labels, threads, &cuda_err, ncap)
                  : o.store_rank == 0
                      ? ctx->store.init_shared(n, row_ptr, col, labels, threads, &cuda_err, o.store_world)
                      : ctx->store.attach_shared(o.store_handle, n, threads, &cuda_err, o.store_rank, o.store_world);
  ctx->opt.store_handle = nullptr;  // caller-owned: not kept
  if (!e.empty()) {
    if (std::getenv("GCSM_TRACE")) std::fprintf(stderr, "[gcsm] create: %s\n", e.c_str());
    delete ctx;
    return cuda_err ? GCSM_EDEVICE : GCSM_EINVAL;
  }
  auto bail = [&](gcsm_status s) {
    delete ctx;
    return s;
  };
  if (cudaStreamCreateWithFlags(&ctx->stream, cudaStreamNonBlocking) != cudaSuccess) return bail(GCSM_EDEVICE);
  if (cudaStreamCreateWithFlags(&ctx->stream2, cudaStreamNonBlocking) != cudaSuccess) return bail(GCSM_EDEVICE);
  {  // the cache step's stream takes the higher scheduling priority (it feeds the next batch's matching): its blocks
     // go first when the extension kernels' blocks retire (GCSM_CS_PRIO=0: default priority; A/B in
     // profiles/ab_r01_reserve.txt)
    int lo = 0, hi = 0;
    cudaDeviceGetStreamPriorityRange(&lo, &hi);
    const char *pe = std::getenv("GCSM_CS_PRIO");
    const int prio = (pe && std::atoi(pe) == 0) ? lo : hi;
    if (cudaStreamCreateWithPriority(&ctx->stream3, cudaStreamNonBlocking, prio) != cudaSuccess) return bail(GCSM_EDEVICE);
  }
  for (auto &sl : ctx->slots) {
    for (cudaEvent_t *ev : {&sl.ev_a0, &sl.ev_a1, &sl.ev_c0, &sl.ev_c1, &sl.ev_done})
      if (cudaEventCreate(ev) != cudaSuccess) return bail(GCSM_EDEVICE);
    for (cudaEvent_t *ev : {&sl.ev_up, &sl.ev_l2})
      if (cudaEventCreateWithFlags(ev, cudaEventDisableTiming) != cudaSuccess) return bail(GCSM_EDEVICE);
    if (cudaHostAlloc(&sl.h_cnt, sizeof(unsigned long long) * CNT_N * GCSM_MAX_QUERIES, cudaHostAllocDefault) !=
        cudaSuccess)
      return bail(GCSM_ENOMEM);
  }
  for (auto &sl : ctx->slots)
    if (cudaMalloc(&sl.d_vdesc, sizeof(VDesc) * (size_t)ncap) != cudaSuccess ||
        cudaMalloc(&sl.d_cnt, sizeof(unsigned long long) * CNT_N * GCSM_MAX_QUERIES) != cudaSuccess)
      return bail(GCSM_ENOMEM);
  if (cudaMalloc(&ctx->d_hist, sizeof(uint32_t) * (size_t)ncap) != cudaSuccess) return bail(GCSM_ENOMEM);
  if (cudaMalloc(&ctx->d_bsum, sizeof(uint32_t) * (((size_t)ncap + 2047) / 2048 + 1)) != cudaSuccess)
    return bail(GCSM_ENOMEM);
  {
    std::vector<VDesc> vd(ncap, VDesc{nullptr, 0, 0});  // ids [n, ncap): empty until they join
    for (int32_t v = 0; v < n; ++v) vd[v] = VDesc{ctx->store.dev_ptr(ctx->store.lst[v]), ctx->store.len[v], 0};
    for (auto &sl : ctx->slots)
      if (cudaMemcpy(sl.d_vdesc, vd.data(), sizeof(VDesc) * (size_t)ncap, cudaMemcpyHostToDevice) != cudaSuccess)
        return bail(GCSM_EDEVICE);
  }
  if (!ctx->store.lab.empty()) {
    if (cudaMalloc(&ctx->d_lab, 2 * (size_t)ncap) != cudaSuccess) return bail(GCSM_ENOMEM);
    if (cudaMemcpy(ctx->d_lab, ctx->store.lab.data(), 2 * (size_t)ncap, cudaMemcpyHostToDevice) != cudaSuccess)
      return bail(GCSM_EDEVICE);
  }
  ctx->mark.assign(ncap, 0);
  ctx->slot16.assign(ncap, 0);
  for (int q = 0; q < GCSM_MAX_QUERIES; ++q) ctx->lev_levels[q] = -1;
  if (const char *he = std::getenv("GCSM_HOST_EST")) ctx->gpu_est = std::atoi(he) == 0;
  ctx->overlap = ctx->gpu_est && !std::getenv("GCSM_NO_OVERLAP");
  if (const char *ok = std::getenv("GCSM_OVERLAP_KMAX")) ctx->overlap_kmax = std::atoi(ok);
  if (const char *sm = std::getenv("GCSM_STAGE_MB")) ctx->opt.staging_bytes = std::strtoull(sm, nullptr, 10) << 20;
  if (const char *sm = std::getenv("GCSM_STAGE_MIN")) ctx->stage_min = (uint32_t)std::max(1, std::atoi(sm));
  if (const char *sp = std::getenv("GCSM_STAGE_POLICY")) ctx->stage_policy = std::atoi(sp);
  if (const char *ws = std::getenv("GCSM_WALK_STAGE")) ctx->walk_stage = std::atoi(ws);
  if (const char *wl = std::getenv("GCSM_WALK_LANE")) ctx->walk_lane = std::atoi(wl);
  if (std::getenv("GCSM_BCOMP") && gcsm_set_measure(ctx, GCSM_MEASURE_BCOMP) != GCSM_OK) return bail(GCSM_ENOMEM);
  ctx->grid = match_grid(dev, &ctx->warps_total);
  ctx->ext_grid = ctx->grid;
  if (const char *r = std::getenv("GCSM_EXT_RESERVE"))
    if (ctx->overlap) ctx->ext_grid = std::max(1, ctx->grid - std::atoi(r));
  // a communicator whenever an id is given (world 1 included: the single-rank allreduce exercises the same path)
  // (created at the first batch, which every rank enters collectively: creating it here would block rank 0 of a
  // node-shared store in ncclCommInitRank before the other ranks could attach to the store it just made)
  if (o.nccl_id && !(o.flags & GCSM_FLAG_LOCAL_COUNTS)) {
    std::memcpy(ctx->nccl_id, o.nccl_id, sizeof ctx->nccl_id);
    ctx->comm_pending = true;
  }
  ctx->opt.nccl_id = nullptr;  // caller-owned: copied
  *out = ctx;
  return GCSM_OK;
}

void gcsm_destroy(gcsm_ctx *ctx) { delete ctx; }

int32_t gcsm_num_vertices(const gcsm_ctx *ctx) { return ctx ? ctx->store.n : 0; }

gcsm_status gcsm_link_peers(gcsm_ctx *const *ctxs, int32_t n) {
  if (n < 0 || n > GCSM_MAX_PEERS + 1 || (n > 0 && !ctxs)) return GCSM_EINVAL;
  for (int32_t i = 0; i < n; ++i) {
    if (!ctxs[i]) return GCSM_EINVAL;
    if (ctxs[i]->poisoned) return GCSM_ESTATE;
    if (ctxs[i]->waited != ctxs[i]->batch_seq) return ctxs[i]->fail(GCSM_ESTATE, "link_peers with a batch in flight");
    for (int32_t j = 0; j < i; ++j)
      if (ctxs[j] == ctxs[i]) return GCSM_EINVAL;
    if (ctxs[i]->store.ncap != ctxs[0]->store.ncap || ctxs[i]->batch_seq != ctxs[0]->batch_seq)
      return ctxs[i]->fail(GCSM_EINVAL, "linked contexts need the same vertex capacity and batch count");
  }
  for (int32_t i = 0; i < n; ++i) peer_leave(ctxs[i]);
  if (n < 2) return GCSM_OK;
  for (int32_t i = 0; i < n; ++i)  // peer access between distinct devices (NVLink through NVSwitch)
    for (int32_t j = 0; j < n; ++j) {
      const int di = ctxs[i]->device, dj = ctxs[j]->device;
      if (di == dj) continue;
      int can = 0;
      cudaDeviceCanAccessPeer(&can, di, dj);
      if (!can) return ctxs[i]->fail(GCSM_EDEVICE, "no peer access between the linked devices");
      cudaSetDevice(di);
      const cudaError_t e = cudaDeviceEnablePeerAccess(dj, 0);
      if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled) return ctxs[i]->cuda_fail(e, "peer access");
      cudaGetLastError();
    }
  auto pg = std::make_shared<PeerGroup>();
  pg->members.assign(ctxs, ctxs + n);
  pg->enq.assign((size_t)n, ctxs[0]->batch_seq);
  for (int32_t i = 0; i < n; ++i) {
    ctxs[i]->peers = pg;
    ctxs[i]->peer_idx = i;
    cudaSetDevice(ctxs[i]->device);
  }
  return GCSM_OK;
}

gcsm_status gcsm_link_store_peers(gcsm_ctx *ctx) {
  if (!ctx) return GCSM_EINVAL;
  if (ctx->poisoned) return GCSM_ESTATE;
  HostStore &S = ctx->store;
  if (!S.shared()) return ctx->fail(GCSM_EINVAL, "gcsm_link_store_peers needs a node-shared store");
  if (ctx->waited != ctx->batch_seq) return ctx->fail(GCSM_ESTATE, "link with a batch in flight");
  if (ctx->sp.n) return ctx->fail(GCSM_ESTATE, "already linked");
  if (!ctx->d_cachebuf[0] || !ctx->d_cachebuf[1]) return ctx->fail(GCSM_ESTATE, "set the cache budget first");
  if (S.store_world() - 1 > GCSM_MAX_PEERS) return ctx->fail(GCSM_EINVAL, "too many peers");
  cudaSetDevice(ctx->device);
  for (cudaEvent_t &e : ctx->ev_ipc)
    if (!e) CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming | cudaEventInterprocess));
  PeerMail *me = reinterpret_cast<PeerMail *>(S.mailbox(S.store_rank()));
  std::memset((void *)me, 0, sizeof *me);
  for (int j = 0; j < 2; ++j) {
    CK(cudaIpcGetMemHandle(&me->cache[j], ctx->d_cachebuf[j]));
    CK(cudaIpcGetMemHandle(&me->vdesc[j], ctx->slots[j].d_vdesc));
    CK(cudaIpcGetEventHandle(&me->ev[j], ctx->ev_ipc[j]));
    me->cache_va[j] = (uint64_t)(uintptr_t)ctx->d_cachebuf[j];
    me->cache_idx[j] = -1;
  }
  me->cache_cap = ctx->cache_cap;
  me->device = ctx->device;
  me->linked = 1;
  if (!S.barrier()) return ctx->fail(GCSM_ESTATE, S.shared_err);
  StorePeers sp;
  bool ok = true;
  for (int r = 0; r < S.store_world() && ok; ++r) {
    if (r == S.store_rank()) continue;
    const PeerMail *pm = reinterpret_cast<const PeerMail *>(S.mailbox(r));
    if (!pm->linked) {
      ok = false;
      break;
    }
    const int p = sp.n++;
    sp.rank[p] = r;
    sp.cache_cap[p] = pm->cache_cap;
    for (int j = 0; j < 2 && ok; ++j) {
      sp.cache_va[p][j] = pm->cache_va[j];
      ok = cudaIpcOpenMemHandle(&sp.vdesc[p][j], pm->vdesc[j], cudaIpcMemLazyEnablePeerAccess) == cudaSuccess &&
           cudaIpcOpenMemHandle((void **)&sp.cache_map[p][j], pm->cache[j], cudaIpcMemLazyEnablePeerAccess) ==
               cudaSuccess &&
           cudaIpcOpenEventHandle(&sp.ev[p][j], pm->ev[j]) == cudaSuccess;
    }
  }
  ctx->sp = sp;
  if (!ok) {
    cudaGetLastError();
    store_peers_close(ctx);
    S.poison_shared();
    return ctx->fail(GCSM_EDEVICE, "opening a peer's IPC handles failed");
  }
  if (!S.barrier()) return ctx->fail(GCSM_ESTATE, S.shared_err);
  return GCSM_OK;
}

gcsm_status gcsm_store_handle(const gcsm_ctx *ctx, char *buf, uint64_t cap) {
  if (!ctx || !buf || !ctx->store.shared() || ctx->store.store_rank() != 0) return GCSM_EINVAL;
  const std::string h = ctx->store.handle();
  if (cap < h.size() + 1) return GCSM_EINVAL;
  std::memcpy(buf, h.c_str(), h.size() + 1);
  return GCSM_OK;
}

gcsm_status gcsm_add_vertices(gcsm_ctx *ctx, int32_t count, const int32_t *labels, int32_t *first_id) {
  if (!ctx || count < 0) return GCSM_EINVAL;
  if (ctx->poisoned) return GCSM_ESTATE;
  if (ctx->waited != ctx->batch_seq) return ctx->fail(GCSM_ESTATE, "add_vertices with a batch in flight");
  HostStore &S = ctx->store;
  if ((int64_t)S.n + count > (int64_t)S.ncap) return ctx->fail(GCSM_EINVAL, "vertex capacity exceeded");
  if (labels) {
    if (S.lab.empty()) return ctx->fail(GCSM_EINVAL, "labels for new vertices of an unlabelled graph");
    for (int32_t i = 0; i < count; ++i)
      if (labels[i] < 0 || labels[i] > 65535) return ctx->fail(GCSM_EINVAL, "label out of [0, 65535]");
  }
  const int32_t first = S.n;
  if (!S.grow(S.n + count)) return ctx->fail(GCSM_ENOMEM, "pinned allocation for new vertices failed");
  if (labels) {
    for (int32_t i = 0; i < count; ++i) S.lab[first + i] = (uint16_t)labels[i];
    if (ctx->d_lab) {
      if (cudaSetDevice(ctx->device) != cudaSuccess) return ctx->fail(GCSM_EDEVICE, "cudaSetDevice");
      CK(cudaMemcpy(ctx->d_lab + first, S.lab.data() + first, 2 * (size_t)count, cudaMemcpyHostToDevice));
    }
  }
  if (first_id) *first_id = first;
  ctx->err.clear();
  return GCSM_OK;
}

gcsm_status gcsm_set_measure(gcsm_ctx *ctx, uint32_t flags) {
  if (!ctx || (flags & ~(uint32_t)GCSM_MEASURE_BCOMP)) return GCSM_EINVAL;
  if (ctx->poisoned) return GCSM_ESTATE;
  const bool on = (flags & GCSM_MEASURE_BCOMP) != 0;
  if (on && !ctx->d_touched_bc) {
    if (cudaSetDevice(ctx->device) != cudaSuccess) return GCSM_EDEVICE;
    if (cudaMalloc(&ctx->d_touched_bc, 4 * (((size_t)ctx->store.ncap + 31) / 32)) != cudaSuccess) {
      cudaGetLastError();
      ctx->d_touched_bc = nullptr;
      return GCSM_ENOMEM;
    }
  }
  ctx->bcomp = on;
  return GCSM_OK;
}

const char *gcsm_last_error(const gcsm_ctx *ctx) { return ctx ? ctx->err.c_str() : "null context"; }

gcsm_status gcsm_get_stream(const gcsm_ctx *ctx, void **stream) {
  if (!ctx || !stream) return GCSM_EINVAL;
  *stream = (void *)ctx->stream;
  return GCSM_OK;
}

static gcsm_status add_query_impl(gcsm_ctx *ctx, bool reset, int32_t k, int32_t m, const int32_t *qedges,
                                  const int32_t *qlabels, const int32_t *order, int32_t *qid) {
  if (!ctx) return GCSM_EINVAL;
  if (ctx->poisoned) return GCSM_ESTATE;
  if (ctx->waited != ctx->batch_seq) return ctx->fail(GCSM_ESTATE, "set_query / add_query with a batch in flight");
  if (!reset && !ctx->has_query) return ctx->fail(GCSM_ESTATE, "add_query before set_query");
  if (!reset && ctx->qs.size() >= GCSM_MAX_QUERIES) return ctx->fail(GCSM_EINVAL, "too many standing queries");
  gcsm_ctx::Query q;
  std::string e = build_plan(k, m, qedges, qlabels, order, q.qp);
  if (e.empty()) e = build_plan(k, m, qedges, qlabels, order, q.qps, !(ctx->opt.flags & GCSM_FLAG_NO_SYMMETRY));
  if (!e.empty()) return ctx->fail(GCSM_EINVAL, e);
  if (q.qp.labelled && !ctx->d_lab) {  // unlabelled graph: every data label is 0 (R5)
    CK(cudaMalloc(&ctx->d_lab, 2 * (size_t)ctx->store.ncap));
    CK(cudaMemset(ctx->d_lab, 0, 2 * (size_t)ctx->store.ncap));
  }
  const size_t slot = reset ? 0 : ctx->qs.size();
  DevPlan *dp = slot < ctx->qs.size() ? ctx->qs[slot].d_plans : nullptr;
  DevPlan *dsp = slot < ctx->qs.size() ? ctx->qs[slot].d_splans : nullptr;
  if (!dp && cudaMalloc(&dp, sizeof(DevPlan) * GCSM_MAXPLANS) != cudaSuccess)
    return ctx->fail(GCSM_ENOMEM, "plan buffer");
  if (!dsp && cudaMalloc(&dsp, sizeof(DevPlan) * GCSM_MAXPLANS) != cudaSuccess) {
    if (slot >= ctx->qs.size()) cudaFree(dp);
    return ctx->fail(GCSM_ENOMEM, "plan buffer");
  }
  q.d_plans = dp;
  q.d_splans = dsp;
  CK(upload_plans(dp, q.qp.plans.data(), (int)q.qp.plans.size(), ctx->stream));
  CK(upload_plans(dsp, q.qps.plans.data(), (int)q.qps.plans.size(), ctx->stream));
  CK(cudaStreamSynchronize(ctx->stream));
  if (reset)
    for (int &l : ctx->lev_levels) l = -1;  // walk sums of other patterns are stale: re-zeroed on next use
  else
    ctx->lev_levels[slot] = -1;
  if (reset) {
    for (size_t i = 1; i < ctx->qs.size(); ++i) {
      cudaFree(ctx->qs[i].d_plans);
      cudaFree(ctx->qs[i].d_splans);
    }
    ctx->qs.clear();
  }
  ctx->qs.push_back(std::move(q));
  if (qid) *qid = (int32_t)ctx->qs.size() - 1;
  ctx->has_query = true;
  ctx->err.clear();
  return GCSM_OK;
}

gcsm_status gcsm_set_query(gcsm_ctx *ctx, int32_t k, int32_t m, const int32_t *qedges, const int32_t *qlabels,
                           const int32_t *order) {
  return add_query_impl(ctx, true, k, m, qedges, qlabels, order, nullptr);
}

gcsm_status gcsm_add_query(gcsm_ctx *ctx, int32_t k, int32_t m, const int32_t *qedges, const int32_t *qlabels,
                           const int32_t *order, int32_t *qid) {
  return add_query_impl(ctx, false, k, m, qedges, qlabels, order, qid);
}

int32_t gcsm_num_queries(const gcsm_ctx *ctx) { return ctx && ctx->has_query ? (int32_t)ctx->qs.size() : 0; }

gcsm_status gcsm_set_cache_budget(gcsm_ctx *ctx, uint64_t bytes) {
  if (!ctx) return GCSM_EINVAL;
  if (ctx->poisoned) return GCSM_ESTATE;
  if (ctx->waited != ctx->batch_seq) return ctx->fail(GCSM_ESTATE, "set_cache_budget with a batch in flight");
  bytes &= ~uint64_t(15);
  if (ctx->sp.n && bytes > ctx->cache_cap)  // the peers hold IPC mappings of the current buffers
    return ctx->fail(GCSM_EINVAL, "a store-peer-linked cache cannot grow");
  if (bytes > ctx->cache_cap) {
    for (char *&b : ctx->d_cachebuf) {
      if (b) cudaFree(b);
      b = nullptr;
    }
    ctx->cache_cap = 0;
    for (char *&b : ctx->d_cachebuf)
      if (cudaMalloc(&b, bytes) != cudaSuccess) return ctx->fail(GCSM_ENOMEM, "device cache allocation failed");
    ctx->cache_cap = bytes;
  }
  ctx->budget = bytes;
  ctx->cache_valid = false;  // the next batch repacks everything
  for (int32_t v : ctx->prev_cached) ctx->slot16[v] = 0;
  ctx->cache_reset = true;   // GPU packer: the previous selection's descriptors may point into a freed buffer
  return GCSM_OK;
}

}  // extern "C"

// ------------------------------------------------------------------ pipeline

// Merge of two id-ascending (score, id) lists, summing the scores of common ids; parallel over id ranges.
static std::vector<std::pair<double, int32_t>> merge_sum_by_id(const std::vector<std::pair<double, int32_t>> &x,
                                                              const std::vector<std::pair<double, int32_t>> &y,
                                                              int T) {
  const int nt = std::max(1, std::min(T, pool_size()));
  const int64_t lo_id = std::min(x.empty() ? INT32_MAX : x.front().second, y.empty() ? INT32_MAX : y.front().second);
  const int64_t hi_id = std::max(x.empty() ? 0 : x.back().second, y.empty() ? 0 : y.back().second) + 1;
  std::vector<int64_t> cut(nt + 1);
  for (int t = 0; t <= nt; ++t) cut[t] = lo_id + (hi_id - lo_id) * t / nt;
  auto lb = [](const std::vector<std::pair<double, int32_t>> &v, int64_t id) {
    return (size_t)(std::lower_bound(v.begin(), v.end(), id,
                                     [](const std::pair<double, int32_t> &e, int64_t k) { return e.second < k; }) -
                    v.begin());
  };
  std::vector<std::vector<std::pair<double, int32_t>>> part(nt);
  parallel_for(nt, nt, [&](int, int64_t t0, int64_t t1) {
    for (int64_t t = t0; t < t1; ++t) {
      size_t i = lb(x, cut[t]), ie = lb(x, cut[t + 1]), j = lb(y, cut[t]), je = lb(y, cut[t + 1]);
      auto &o = part[t];
      o.reserve((ie - i) + (je - j));
      while (i < ie || j < je) {
        if (j == je || (i < ie && x[i].second < y[j].second)) o.push_back(x[i++]);
        else if (i == ie || y[j].second < x[i].second) o.push_back(y[j++]);
        else {
          o.push_back({x[i].first + y[j].first, x[i].second});
          ++i;
          ++j;
        }
      }
    }
  });
  std::vector<std::pair<double, int32_t>> out;
  size_t tot = 0;
  for (auto &p : part) tot += p.size();
  out.reserve(tot);
  for (auto &p : part) out.insert(out.end(), p.begin(), p.end());
  return out;
}

static uint16_t host_label(const HostStore &s, int32_t v) { return s.lab.empty() ? 0 : s.lab[v]; }

// GCSM_TRACE=1: per-batch host sub-step timings on stderr (development aid).
struct Trace {
  bool on = std::getenv("GCSM_TRACE") != nullptr;
  Timer t;
  double last = 0;
  std::string line;
  void mark(const char *name) {
    if (!on) return;
    const double now = t.ms();
    char buf[64];
    std::snprintf(buf, sizeof buf, " %s=%.2f", name, now - last);
    line += buf;
    last = now;
  }
  ~Trace() {
    if (on) std::fprintf(stderr, "[gcsm trace]%s\n", line.c_str());
  }
};

// GPU path of steps (2)-(3) (estimator_gpu.cu): uploads the batch's delta records, units, changed descriptors (host
// addresses) and level-1 walk nodes, then enqueues the walks, the ranking cut and the cache copy on the stream.
static gcsm_status enqueue_gpu_cache(gcsm_ctx *ctx, gcsm_ctx::Slot &sl, cudaStream_t s, size_t ndirty, size_t nU,
                                     size_t nd, int64_t gnu, const std::vector<std::vector<EstUnit>> &qeu,
                                     const std::vector<std::vector<int2>> &qitems, const std::vector<int64_t> &qf2cap,
                                     uint64_t maxB, uint64_t D, const std::vector<int64_t> &qnu,
                                     const std::vector<uint64_t> &qwalks, bool use_cache, uint64_t *launches) {
  HostStore &S = ctx->store;
  const int32_t n = S.n;
  const int nq = (int)ctx->qs.size();
  if (!ctx->gpu_ready) {  // n-sized buffers at the vertex capacity (ids may grow into it)
    const int32_t nc = S.ncap;
    const size_t W = ((size_t)nc + 31) / 32 + 1;
    std::vector<unsigned long long> hp((size_t)nc, 0ull);
    for (int32_t v = 0; v < n; ++v) hp[v] = (unsigned long long)(uintptr_t)S.dev_ptr(S.lst[v]);
    ctx->cubtmp_bytes = cache_step_tmp_bytes(nc);
    if (cudaMalloc(&ctx->d_hptr, 8 * (size_t)nc) != cudaSuccess || cudaMalloc(&ctx->d_touched, 4 * W) != cudaSuccess ||
        cudaMalloc(&ctx->d_wcnt, 4 * W) != cudaSuccess || cudaMalloc(&ctx->d_woff, 4 * W) != cudaSuccess ||
        cudaMalloc(&ctx->d_tids, 4 * (size_t)nc) != cudaSuccess || cudaMalloc(&ctx->d_prev_sel, 4 * (size_t)nc) != cudaSuccess ||
        cudaMalloc(&ctx->d_bits, 8 * (size_t)nc) != cudaSuccess || cudaMalloc(&ctx->d_bytes, 8 * (size_t)nc) != cudaSuccess ||
        cudaMalloc(&ctx->d_scan, 8 * (size_t)nc) != cudaSuccess || cudaMalloc(&ctx->d_off, 8 * (size_t)nc) != cudaSuccess ||
        cudaMalloc(&ctx->d_flag, (size_t)nc) != cudaSuccess ||
        cudaMalloc(&ctx->d_selhist, 8 * 6 * 4096) != cudaSuccess ||
        cudaMalloc(&ctx->d_ecursor, 8 * 3 * GCSM_MAX_QUERIES) != cudaSuccess ||
        cudaMalloc(&ctx->d_sel, sizeof(SelState)) != cudaSuccess ||
        cudaMalloc(&ctx->d_cubtmp, ctx->cubtmp_bytes) != cudaSuccess)
      return ctx->fail(GCSM_ENOMEM, "GPU estimator buffers");
    CK(cudaMemcpyAsync(ctx->d_hptr, hp.data(), 8 * (size_t)nc, cudaMemcpyHostToDevice, s));
    double sfc[10];
    for (int i = 0; i < 10; ++i) sfc[i] = stirling_small(i);
    if (cudaMalloc(&ctx->d_sfc, sizeof sfc) != cudaSuccess) return ctx->fail(GCSM_ENOMEM, "GPU estimator buffers");
    CK(cudaMemcpyAsync(ctx->d_sfc, sfc, sizeof sfc, cudaMemcpyHostToDevice, s));
    {  // sampled index of every list of >= 64 elements
      ctx->soff_h.assign((size_t)nc, 0xffffffffu);
      ctx->scap_h.assign((size_t)nc, 0);
      size_t total = 0;
      for (int32_t v = 0; v < n; ++v)
        if (S.len[v] >= 64) {
          const uint32_t ns = (S.len[v] + 31) / 32;
          ctx->soff_h[v] = (uint32_t)total;
          ctx->scap_h[v] = ns + 1;
          total += ns + 1;
        }
      ctx->sidx_capacity = total + total / 2 + ((size_t)1 << 20);
      ctx->sidx_next = total;
      std::vector<int32_t> smp(total);
      parallel_for(ctx->opt.host_threads, n, [&](int, int64_t lo, int64_t hi) {
        for (int64_t v = lo; v < hi; ++v)
          if (ctx->soff_h[v] != 0xffffffffu)
            for (uint32_t j = 0; 32 * j < S.len[v]; ++j) smp[ctx->soff_h[v] + j] = S.lst[v][32 * j];
      });
      if (ctx->sidx_capacity >= ((size_t)1 << 31) || cudaMalloc(&ctx->d_sidx, 4 * ctx->sidx_capacity) != cudaSuccess ||
          cudaMalloc(&ctx->d_soff, 4 * (size_t)nc) != cudaSuccess)
        return ctx->fail(GCSM_ENOMEM, "sampled list index");
      CK(cudaMemcpyAsync(ctx->d_sidx, smp.data(), 4 * total, cudaMemcpyHostToDevice, s));
      CK(cudaMemcpyAsync(ctx->d_soff, ctx->soff_h.data(), 4 * (size_t)nc, cudaMemcpyHostToDevice, s));
      CK(cudaStreamSynchronize(s));  // pageable sources
    }
    CK(cudaMemsetAsync(ctx->d_sel, 0, sizeof(SelState), s));
    CK(cudaStreamSynchronize(s));  // hp is pageable and local
    ctx->gpu_ready = true;
  }
  const bool est_on = use_cache && ctx->opt.cache_policy == GCSM_CACHE_ESTIMATOR;
  for (int qi = 0; qi < nq; ++qi) {  // dense per-vertex walk sums (zero outside the last touched set)
    const int L = ctx->qs[qi].qp.k - 2;
    if (L <= 0 || ctx->lev_levels[qi] == L) continue;
    if (ctx->d_levcnt[qi]) cudaFree(ctx->d_levcnt[qi]);
    ctx->d_levcnt[qi] = nullptr;
    if (cudaMalloc(&ctx->d_levcnt[qi], 8 * (size_t)S.ncap * L) != cudaSuccess)
      return ctx->fail(GCSM_ENOMEM, "estimator sums");
    CK(cudaMemsetAsync(ctx->d_levcnt[qi], 0, 8 * (size_t)S.ncap * L, s));
    ctx->lev_levels[qi] = L;
  }
  // binomial tables: BINV's r0 = (1 - 1/D)^n (host pow, as the host walker computes it) for n up to the largest
  // level-1 multiplicity inside BINV's domain n p < 10 (children draw with n <= their parent's B); rebuilt when
  // D changes or the batch needs more entries, staged in this slot's pinned buffer and copied on the stream
  const double pD = 1.0 / (double)D;
  if (est_on) {
    int64_t nlim = (int64_t)std::ceil(10.0 / pD) + 2;
    while (nlim > 0 && (double)nlim * pD >= 10.0) --nlim;
    const size_t need = (size_t)std::min<int64_t>((int64_t)maxB, nlim) + 1;
    if (pD != ctx->r0_pD || need > ctx->r0_n) {
      const size_t want = std::min<size_t>((size_t)nlim + 1, std::max<size_t>(2 * need, 4096));
      if (!host_ensure(sl.h_r0, sl.h_r0_cap, want)) return ctx->fail(GCSM_ENOMEM, "r0 table");
      double *h = sl.h_r0;
      parallel_for(ctx->opt.host_threads, (int64_t)want, [&](int, int64_t lo, int64_t hi) {
        for (int64_t i = lo; i < hi; ++i) h[i] = std::pow(1.0 - pD, (double)i);
      });
      if (!dev_ensure(ctx->d_r0, ctx->r0_cap, want)) return ctx->fail(GCSM_ENOMEM, "r0 table");
      CK(cudaMemcpyAsync(ctx->d_r0, h, 8 * want, cudaMemcpyHostToDevice, s));
      ctx->r0_pD = pD;
      ctx->r0_n = want;
    }
  }
  // uploads
  size_t neu = 0, nit = 0;
  int64_t f2max = 0;
  for (const auto &eu : qeu) neu += eu.size();
  for (const auto &it : qitems) nit += it.size();
  for (int64_t c2 : qf2cap) f2max = std::max(f2max, c2);
  if (!host_ensure(sl.h_eunits, sl.h_eunits_cap, neu) || !dev_ensure(ctx->d_eunits, ctx->eunits_cap, neu) ||
      !host_ensure(sl.h_eitems, sl.h_eitems_cap, nit) || !dev_ensure(ctx->d_eitems, ctx->eitems_cap, nit) ||
      (f2max > 0 && !dev_ensure(ctx->d_ef2, ctx->ef2_cap, (size_t)f2max)))
    return ctx->fail(GCSM_ENOMEM, "walk roots");
  {
    size_t o = 0, oi = 0;
    for (int qi = 0; qi < nq; ++qi) {
      if (!qeu[qi].empty()) std::memcpy(sl.h_eunits + o, qeu[qi].data(), sizeof(EstUnit) * qeu[qi].size());
      if (!qitems[qi].empty()) std::memcpy(sl.h_eitems + oi, qitems[qi].data(), sizeof(int2) * qitems[qi].size());
      o += qeu[qi].size();
      oi += qitems[qi].size();
    }
  }
  CK(cudaMemsetAsync(sl.d_cnt, 0, sizeof(unsigned long long) * CNT_N * (size_t)nq, s));
  if (sl.ulist_n) CK(cudaMemcpyAsync(sl.d_ulist, sl.h_ulist, 4 * sl.ulist_n, cudaMemcpyHostToDevice, s));
  if (nU) CK(cudaMemcpyAsync(sl.d_drec, sl.h_drec, sizeof(DRec) * nU, cudaMemcpyHostToDevice, s));
  if (nd) CK(cudaMemcpyAsync(sl.d_dlist, sl.h_dlist, 4 * nd, cudaMemcpyHostToDevice, s));
  if (gnu) CK(cudaMemcpyAsync(sl.d_units, sl.h_units, sizeof(Unit) * (size_t)gnu, cudaMemcpyHostToDevice, s));
  if (neu) CK(cudaMemcpyAsync(ctx->d_eunits, sl.h_eunits, sizeof(EstUnit) * neu, cudaMemcpyHostToDevice, s));
  if (nit) CK(cudaMemcpyAsync(ctx->d_eitems, sl.h_eitems, sizeof(int2) * nit, cudaMemcpyHostToDevice, s));
  {  // the previous batch's updated vertices were merged into new lists: refresh their samples
    const std::vector<int32_t> &pu = ctx->prev_U;
    size_t nst = 0;
    for (int32_t v : pu)
      if (S.len[v] >= 64) nst += (S.len[v] + 31) / 32;
    if (!pu.empty()) {
      if (!host_ensure(sl.h_srec, sl.h_srec_cap, pu.size()) || !host_ensure(sl.h_sstage, sl.h_sstage_cap, nst + 1) ||
          !dev_ensure(ctx->d_srec, ctx->srec_cap, pu.size()) || !dev_ensure(ctx->d_sstage, ctx->sstage_cap, nst + 1))
        return ctx->fail(GCSM_ENOMEM, "sampled index staging");
      size_t pos = 0;
      for (size_t i = 0; i < pu.size(); ++i) {
        const int32_t v = pu[i];
        int32_t off = -1, ns = 0;
        if (S.len[v] >= 64) {
          ns = (int32_t)((S.len[v] + 31) / 32);
          if ((uint32_t)ns <= ctx->scap_h[v] && ctx->soff_h[v] != 0xffffffffu) {
            off = (int32_t)ctx->soff_h[v];
          } else if (ctx->sidx_next + 2 * (size_t)ns <= ctx->sidx_capacity) {
            off = (int32_t)ctx->sidx_next;
            ctx->scap_h[v] = 2 * (uint32_t)ns;
            ctx->sidx_next += 2 * (size_t)ns;
          }
          if (off >= 0)
            for (int32_t j = 0; j < ns; ++j) sl.h_sstage[pos + j] = S.lst[v][32 * j];
        }
        if (off < 0) ctx->scap_h[v] = 0;
        ctx->soff_h[v] = off >= 0 ? (uint32_t)off : 0xffffffffu;
        sl.h_srec[i] = int4{v, off, off >= 0 ? ns : 0, (int)pos};
        if (off >= 0) pos += (size_t)ns;
      }
      CK(cudaMemcpyAsync(ctx->d_srec, sl.h_srec, sizeof(int4) * pu.size(), cudaMemcpyHostToDevice, s));
      if (pos) CK(cudaMemcpyAsync(ctx->d_sstage, sl.h_sstage, 4 * pos, cudaMemcpyHostToDevice, s));
      CK(launch_sidx_update(ctx->d_sidx, ctx->d_soff, ctx->d_srec, (int64_t)pu.size(), ctx->d_sstage, s));
      ++*launches;
    }
  }
  if (ndirty) {
    CK(cudaMemcpyAsync(ctx->d_pidx, sl.h_pidx, sizeof(int64_t) * ndirty, cudaMemcpyHostToDevice, s));
    CK(cudaMemcpyAsync(ctx->d_pval, sl.h_pval, sizeof(VDesc) * ndirty, cudaMemcpyHostToDevice, s));
    CK(launch_patch_vdesc_host(sl.d_vdesc, ctx->d_hptr, ctx->d_pidx, ctx->d_pval, (int64_t)ndirty, s));
    ++*launches;
  }
  CK(cudaEventRecord(sl.ev_up, s));  // the batch's data is on the device: the level-2 kernels may start (stream2)
  CacheStep c{};
  c.n = n;
  c.nq = nq;
  size_t o = 0, oi = 0;
  for (int qi = 0; qi < nq; ++qi) {
    EstQuery &q = c.q[qi];
    const int k = ctx->qs[qi].qp.k;
    q.plans = ctx->qs[qi].d_plans;
    q.units = ctx->d_eunits + o;
    q.n_units = est_on ? (int64_t)qeu[qi].size() : 0;
    q.items = ctx->d_eitems + oi;
    q.n_items = est_on ? (int64_t)qitems[qi].size() : 0;
    q.f2_cap = qf2cap[qi];
    o += qeu[qi].size();
    oi += qitems[qi].size();
    q.levcnt = k > 2 ? ctx->d_levcnt[qi] : nullptr;
    q.k = k;
    q.N1 = (uint64_t)std::max<int64_t>(qnu[qi], 1);
    q.M = std::max<uint64_t>(qwalks[qi], 1);
    for (int l = 0; l < 8; ++l) q.powD[l] = std::pow((double)D, (double)l);
  }
  c.policy = use_cache ? (ctx->opt.cache_policy == GCSM_CACHE_DEGREE ? 2 : 1) : 0;
  c.reset_first = ctx->cache_reset;
  ctx->cache_reset = false;
  c.budget = ctx->budget;
  c.vdesc = sl.d_vdesc;
  c.hptr = ctx->d_hptr;
  c.drec = sl.d_drec;
  c.dlist = sl.d_dlist;
  c.lab = ctx->d_lab;
  c.pD = pD;
  c.r0tab = ctx->d_r0;
  c.r0n = (int64_t)ctx->r0_n;
  c.sfc_dev = ctx->d_sfc;
  c.touched = ctx->d_touched;
  c.wcnt = ctx->d_wcnt;
  c.woff = ctx->d_woff;
  c.tids = ctx->d_tids;
  c.bits = ctx->d_bits;
  c.bytes = ctx->d_bytes;
  c.scan = ctx->d_scan;
  c.off = ctx->d_off;
  c.flag = ctx->d_flag;
  c.prev_sel = ctx->d_prev_sel;
  c.hist = ctx->d_selhist;
  c.st = ctx->d_sel;
  c.cursor = ctx->d_ecursor;
  c.f2 = ctx->d_ef2;
  c.cub_tmp = ctx->d_cubtmp;
  c.cub_tmp_bytes = ctx->cubtmp_bytes;
  c.cache = ctx->d_cache;
  c.cnt_cached = sl.d_cnt + CNT_CACHED;
  while (sl.ev_walk.size() < 2 * (size_t)nq) {  // walk timing events (per query)
    cudaEvent_t ev;
    CK(cudaEventCreate(&ev));
    sl.ev_walk.push_back(ev);
  }
  c.ev_walk = sl.ev_walk.data();
  for (int qi = 0; qi < nq && qi < GCSM_MAX_QUERIES; ++qi) c.alg_cnt[qi] = sl.d_cnt + (size_t)qi * CNT_N + CNT_WALG;
  sl.walks_timed = est_on;
  c.walk_lane = ctx->walk_lane;
  // device-resident lists at walk time (the last batch's cache, the batch's U lists): everything else a descriptor
  // points to is the pinned host store, whose membership probes may use the sampled index (ctx->d_sidx)
  c.dev_lo[0] = ctx->cache_valid ? ctx->d_cachebuf[ctx->cache_cur] : nullptr;
  c.dev_hi[0] = c.dev_lo[0] ? c.dev_lo[0] + ctx->cache_cap : nullptr;
  c.dev_lo[1] = reinterpret_cast<const char *>(sl.d_ulist);
  c.dev_hi[1] = reinterpret_cast<const char *>(sl.d_ulist + sl.ulist_n);
  if (!std::getenv("GCSM_NO_WALK_SIDX")) {
    c.sidx = ctx->d_sidx;
    c.soff = ctx->d_soff;
  }
  if (ctx->walk_stage_epoch && !std::getenv("GCSM_NO_WALK_STAGE")) {  // the walks' zero-copy lists through the arena
    const gcsm_ctx::StageSlot &sg = ctx->stg[ctx->batch_seq & 1];
    c.stage = StageRef{sg.state, sg.arena, sg.cap, sg.bump, ctx->walk_stage_epoch};
    c.stage_min = ctx->stage_min;
    c.walk_stage = ctx->walk_stage;
    c.stage_cnt = sl.d_cnt + CNT_WFILL;  // query 0's block
  }
  CK(launch_cache_step(c, s, launches));
  ctx->est_valid = est_on;
  CK(cudaEventRecord(sl.ev_c1, s));
  if (ctx->sp.n) CK(cudaEventRecord(ctx->ev_ipc[ctx->batch_seq & 1], s));  // store peers wait on it
  return GCSM_OK;
}

// Host steps (1)-(3) of one batch, its GPU work (3)-(4b) enqueued on the stream, and its host merge (5) into
// fresh arrays; returns without waiting for the kernels (gcsm_wait_batch collects the counts).
static gcsm_status submit_impl(gcsm_ctx *ctx, int64_t n_ins, const int32_t *ins, int64_t n_del, const int32_t *del,
                               int32_t *tup_add, uint64_t add_cap, int32_t *tup_rem, uint64_t rem_cap) {
  if (!ctx) return GCSM_EINVAL;
  if (ctx->poisoned) return GCSM_ESTATE;
  if (!ctx->has_query) return ctx->fail(GCSM_ESTATE, "apply_batch before set_query");
  if (ctx->batch_seq - ctx->waited >= 2)
    return ctx->fail(GCSM_ESTATE, "two batches already in flight: gcsm_wait_batch first");
  auto &sl = ctx->slots[ctx->batch_seq & 1];
  const bool listing = tup_add || tup_rem;
  if (listing && ctx->opt.world > 1 && !(ctx->opt.flags & GCSM_FLAG_LOCAL_COUNTS))
    return ctx->fail(GCSM_EINVAL, "list mode is single-GPU");
  if (listing && ctx->qs.size() != 1) return ctx->fail(GCSM_EINVAL, "list mode needs exactly one query");
  Timer total;
  Trace tr;
  struct AllocScope {  // stream-ordered growth for this submit only
    AllocScope(cudaStream_t st, std::vector<void *> *r) {
      g_alloc_stream = st;
      g_retired_pinned = r;
    }
    ~AllocScope() {
      g_alloc_stream = nullptr;
      g_retired_pinned = nullptr;
    }
  };
  const int nq = (int)ctx->qs.size();
  int kmax = 2;
  for (const auto &q : ctx->qs) kmax = std::max(kmax, q.qp.k);
  // one predicate for the cache step's stream and the allocation mode: with the cache step on its own stream
  // (overlap, every standing query within the overlap size limit) buffers grow synchronously; otherwise
  // stream-ordered on the context stream
  const bool two_streams = ctx->overlap && kmax <= ctx->overlap_kmax;
  AllocScope alloc_scope(two_streams ? nullptr : ctx->stream, &ctx->retired_pinned);
  HostStore &S = ctx->store;
  const int T = ctx->opt.host_threads;
  gcsm_stats st{};
  st.batches = ctx->batch_seq + 1;

  // ---- (1) normalise + overlay + units -------------------------------------------------
  Timer t1;
  if (ctx->comm_pending) {  // every rank's first batch: the count allreduce's communicator
    ncclUniqueId id;
    static_assert(sizeof id == sizeof ctx->nccl_id, "ncclUniqueId is 128 bytes");
    std::memcpy(&id, ctx->nccl_id, sizeof id);
    if (ncclCommInitRank(&ctx->comm, ctx->opt.world, id, ctx->opt.rank) != ncclSuccess) {
      ctx->comm = nullptr;
      return ctx->fail(GCSM_ENCCL, "ncclCommInitRank failed");
    }
    ctx->comm_pending = false;
  }
  if (S.shared()) {  // node-shared store: every rank enters the batch (and has collected batch t-2)
    if (!S.barrier()) {
      ctx->poisoned = true;
      return ctx->fail(GCSM_ESTATE, S.shared_err);
    }
    auto &pr = ctx->pending_retired;
    size_t keep = 0;
    for (auto &p : pr) {
      if (p.first + 2 <= ctx->batch_seq) S.recycle(p.second);
      else pr[keep++] = std::move(p);
    }
    pr.resize(keep);
  }
  std::string e = S.normalize(n_ins, ins, n_del, del);
  if (!e.empty()) return ctx->fail(GCSM_EINVAL, e);
  ctx->in_batch = true;
  if (S.grow_n > S.n && !S.grow(S.grow_n))  // new vertices named by the insertions
    return ctx->fail(GCSM_ENOMEM, "pinned allocation for new vertices failed");
  tr.mark("normalize");
  bool cuda_err = false;
  if (!S.build_overlay((int)(ctx->batch_seq & 1), &cuda_err)) {
    if (S.shared()) {
      S.poison_shared();
      ctx->poisoned = true;
      return ctx->fail(GCSM_ESTATE, S.shared_err);
    }
    return ctx->fail(GCSM_EDEVICE, "pinned overlay allocation failed");
  }
  tr.mark("overlay");
  st.n_ins = S.I.size();
  st.n_del = S.D.size();
  st.dropped = S.dropped;
  const uint64_t D = std::max<uint64_t>(1, std::max<uint64_t>(S.maxdeg, S.maxdeg_new));
  std::vector<std::vector<Unit>> qunits((size_t)nq);
  std::vector<int64_t> qnu((size_t)nq, 0);
  for (int qi = 0; qi < nq; ++qi) {
    const QueryPlan &Q = ctx->qs[qi].qp;
    const int k = Q.k;
    std::vector<Unit> &units = qunits[qi];
    // level-1 units: (term, kind, changed edge, orientation) slots enumerated in parallel, then compacted in slot
    // order (deterministic); the cost proxy of a unit is the list lengths its first level reads
    std::vector<uint64_t> cost;
    {
      const int64_t ni = (int64_t)S.I.size(), ndl = (int64_t)S.D.size(), per = 2 * (ni + ndl);
      const int64_t slots = (int64_t)Q.m * per;
      std::vector<Unit> all((size_t)slots);
      std::vector<uint64_t> ac((size_t)slots, 0);  // 0 = filtered out
      parallel_for(T, slots, [&](int, int64_t lo, int64_t hi) {
        for (int64_t sidx = lo; sidx < hi; ++sidx) {
          const int term = (int)(sidx / per);
          int64_t r = sidx % per;
          const int o = (int)(r & 1);
          r >>= 1;
          const int kind = r < ni ? 0 : 1;
          const uint64_t key = kind ? S.D[r - ni] : S.I[r];
          const DevPlan &P = Q.plans[2 * term + kind];
          const int32_t x = (int32_t)(key >> 32), y = (int32_t)(key & 0xffffffffu);
          const int32_t a = o ? y : x, b = o ? x : y;
          if (P.label0 >= 0 && host_label(S, a) != P.label0) continue;
          if (P.label1 >= 0 && host_label(S, b) != P.label1) continue;
          all[sidx] = Unit{a, b, 2 * term + kind, 0};
          uint64_t c = 1;
          if (k > 2) {
            const LevelPlan &L2 = P.lv[2];
            const int32_t f[2] = {a, b};
            for (int bb = 0; bb < L2.nb; ++bb) c += S.view_len(f[L2.bpos[bb]], L2.bview[bb]);
          }
          ac[sidx] = c;
        }
      });
      units.reserve((size_t)slots);
      cost.reserve((size_t)slots);
      for (int64_t sidx = 0; sidx < slots; ++sidx)
        if (ac[sidx]) {
          units.push_back(all[sidx]);
          cost.push_back(ac[sidx]);
        }
    }
    {  // this rank's LPT shard (world > 1), heaviest units first (dynamic scheduling tail): one parallel stable
       // sort by cost serves both
      std::vector<int32_t> rk(units.size());
      std::vector<size_t> idx;
      shard_lpt((int64_t)units.size(), cost.data(), ctx->opt.world, rk.data(), T, &idx);
      std::vector<Unit> u2;
      std::vector<uint64_t> c2;
      u2.reserve(units.size());
      c2.reserve(units.size());
      for (size_t i : idx)
        if (rk[i] == ctx->opt.rank || ctx->opt.world <= 1) {
          u2.push_back(units[i]);
          c2.push_back(cost[i]);
        }
      units.swap(u2);
      cost.swap(c2);
    }

    qnu[qi] = (int64_t)units.size();
  }
  tr.mark("units");
  st.units = st.n1 = (uint64_t)qnu[0];
  st.max_degree = D;
  st.ms_normalize = t1.ms();

  // ---- (2) estimator (per query; one ranking: the sum of the queries' estimated accesses per vertex) -------
  Timer t2;
  std::vector<std::pair<double, int32_t>> ranked;  // (score, id)
  const bool use_cache = ctx->budget > 0 && ctx->opt.cache_policy != GCSM_CACHE_NONE && kmax > 2;
  std::vector<double> qms_est((size_t)nq, 0.0);
  std::vector<uint64_t> qwalks((size_t)nq, 0);
  // GPU path: the level-1 nodes of the walks (a unit, its key of R22 and its draw B_1 ~ Bin(M, 1/N1)) are
  // made here (N1 draws); everything below level 1 runs in k_walks (estimator_gpu.cu)
  std::vector<std::vector<EstUnit>> qeu(ctx->gpu_est ? (size_t)nq : 0);
  std::vector<std::vector<int2>> qitems(ctx->gpu_est ? (size_t)nq : 0);
  std::vector<int64_t> qf2cap((size_t)nq, 0);
  uint64_t eu_maxB = 0;
  if (ctx->gpu_est) {
    for (int qi = 0; qi < nq; ++qi) {
      Timer tq;
      const QueryPlan &Q = ctx->qs[qi].qp;
      const int k = Q.k;
      const int64_t nu = qnu[qi];
      if (k > 2 && nu > 0) {
        const uint64_t M = ctx->opt.walks_override ? ctx->opt.walks_override : walk_budget((uint64_t)nu, D, k);
        qwalks[qi] = M;
        if (ctx->opt.cache_policy == GCSM_CACHE_ESTIMATOR && ctx->budget > 0) {
          const uint64_t seed = qi == 0 ? ctx->opt.seed : rng_chain(ctx->opt.seed, 0x51ull + (uint64_t)qi);
          const uint64_t root = rng_mix(seed);
          const double p1 = 1.0 / (double)nu;
          const std::vector<Unit> &units = qunits[qi];
          std::vector<EstUnit> all((size_t)nu);
          parallel_for(T, nu, [&](int, int64_t lo, int64_t hi) {
            for (int64_t i = lo; i < hi; ++i) {
              const Unit &u = units[i];
              const uint64_t key =
                  rng_chain(rng_chain(rng_chain(rng_chain(rng_chain(root, ctx->batch_seq), (uint64_t)(u.plan >> 1)),
                                                (uint64_t)(u.plan & 1)),
                                      (uint64_t)(uint32_t)u.a),
                            (uint64_t)(uint32_t)u.b);
              const int64_t B = binomial(key, (int64_t)M, p1);
              all[i] = EstUnit{u.a, u.b, u.plan, 0, (unsigned long long)std::max<int64_t>(B, 0), key};
            }
          });
          std::vector<EstUnit> &eu = qeu[qi];
          eu.reserve(all.size());
          for (const EstUnit &x : all)
            if (x.B > 0) {
              eu.push_back(x);
              eu_maxB = std::max<uint64_t>(eu_maxB, x.B);
            }
          // work items: kEstItem driver elements of a unit's level-1 candidate scan each (hubs spread over warps);
          // level-2 node capacity = the sum of the driver lengths (k >= 5)
          std::vector<int2> &items = qitems[qi];
          int64_t cap2 = 0;
          for (size_t i = 0; i < eu.size(); ++i) {
            const LevelPlan &L2 = Q.plans[eu[i].plan].lv[2];
            const int32_t f[2] = {eu[i].a, eu[i].b};
            int64_t dl = INT64_MAX;
            for (int bb = 0; bb < L2.nb; ++bb) dl = std::min<int64_t>(dl, S.view_len(f[L2.bpos[bb]], L2.bview[bb]));
            if (dl == INT64_MAX) dl = 0;
            cap2 += dl;
            for (int64_t st0 = 0; st0 == 0 || st0 < dl; st0 += kEstItem) items.push_back(int2{(int)i, (int)st0});
          }
          qf2cap[qi] = k >= 5 ? cap2 : 0;
        }
      }
      qms_est[qi] = tq.ms();
    }
    tr.mark("walk_roots");
  }
  for (int qi = 0; qi < nq && !ctx->gpu_est; ++qi) {
    Timer tq;
    const QueryPlan &Q = ctx->qs[qi].qp;
    const int k = Q.k;
    const int64_t nu = qnu[qi];
    EstimatorOutput &est = ctx->qs[qi].est;
    est.ids.clear();
    est.levcnt.clear();
    if (k > 2 && nu > 0) {
      const uint64_t M = ctx->opt.walks_override ? ctx->opt.walks_override : walk_budget((uint64_t)nu, D, k);
      qwalks[qi] = M;
      if (ctx->opt.cache_policy == GCSM_CACHE_ESTIMATOR && ctx->budget > 0) {
        EstimatorInput in;
        in.plans = Q.plans.data();
        in.units = qunits[qi].data();
        in.n_units = nu;
        in.N1 = (uint64_t)nu;
        in.D = D;
        in.M = M;
        in.seed = qi == 0 ? ctx->opt.seed : rng_chain(ctx->opt.seed, 0x51ull + (uint64_t)qi);  // own stream per query
        in.batch_seq = ctx->batch_seq;
        in.labels = S.lab.empty() ? nullptr : S.lab.data();
        in.threads = T;
        in.view = [&S](int32_t v, int vw) { return S.view(v, vw); };
        in.n = S.n;
        run_estimator(in, ctx->est_scratch, est);
        tr.mark("walks");
        if (use_cache) {
          std::vector<std::pair<double, int32_t>> r(est.ids.size());
          parallel_for(T, (int64_t)r.size(), [&](int, int64_t lo, int64_t hi) {
            for (int64_t i = lo; i < hi; ++i)
              r[i] = {estimate_value(&est.levcnt[8 * i], k, (uint64_t)nu, D, M), est.ids[i]};
          });
          if (ranked.empty()) {
            ranked.swap(r);
          } else {  // both ascending by id: merge, summing the scores of a vertex both queries access
            ranked = merge_sum_by_id(ranked, r, T);
          }
        }
      }
    }
    qms_est[qi] = tq.ms();
  }
  st.walks = qwalks[0];
  if (use_cache && ctx->opt.cache_policy == GCSM_CACHE_DEGREE && !ctx->gpu_est) {
    ranked.reserve(S.n);
    for (int32_t v = 0; v < S.n; ++v) {
      const uint32_t d = S.view_len(v, VIEW_S);
      if (d) ranked.emplace_back((double)d, v);
    }
  }
  st.ms_estimate = t2.ms();
  tr.mark("score");
  // symmetry breaking (count mode): the kernels walk only the canonical embedding of every Aut_L orbit and the
  // counts are scaled by |Aut_L| (Emb(G') \ Emb(G) is a union of orbits); the estimator above samples the full
  // execution trees of the paper. Seeds violating a restriction between the two seed endpoints are dropped here.
  std::vector<int64_t> uoff((size_t)nq + 1, 0);
  for (int qi = 0; qi < nq; ++qi) {
    const bool sym = !listing && ctx->qs[qi].qps.symmetry;
    std::vector<Unit> &units = qunits[qi];
    if (sym) {
      const QueryPlan &QK = ctx->qs[qi].qps;
      size_t w = 0;
      for (size_t i = 0; i < units.size(); ++i) {
        const int rel = QK.plans[units[i].plan].seed_rel;
        if (rel == 0 || (rel == 1 ? units[i].a < units[i].b : units[i].a > units[i].b)) units[w++] = units[i];
      }
      units.resize(w);
    }
    uoff[qi + 1] = uoff[qi] + (int64_t)units.size();
  }
  const int64_t gnu = uoff[nq];

  // ---- (3) pack the cache + descriptors --------------------------------------------------
  Timer t3;
  std::vector<int32_t> sel;
  std::vector<uint64_t> sel_off;
  uint64_t used = 0;
  // incremental cache (double buffered): a selected vertex whose list is unchanged since it was cached in the
  // previous batch (not updated then, not updated now) is copied HBM -> HBM; only the other lists go through
  // pinned staging and the one H2D DMA.
  std::vector<uint64_t> gather;  // (src offset, dst offset, 16-byte units) per retained list
  std::vector<uint64_t> fresh;   // (src host address, dst offset, 16-byte units) per newly cached list
  uint64_t new_bytes = 0;
  const int tgt = ctx->cache_valid ? 1 - ctx->cache_cur : ctx->cache_cur;
  ctx->d_cache = ctx->d_cachebuf[tgt];
  if (use_cache && !ranked.empty() && !ctx->gpu_est) {
    // x ∈ U: its list is device-resident with the batch only on the GPU path; the host path keeps the paper's
    // ranking over every vertex (R32)
    // Only the head of the ranking can fit the budget: bucket the (positive) scores by the top 12 bits of their
    // IEEE pattern (monotone in the score), then the next 12 inside the bucket where the cumulative list bytes
    // pass the budget, and sort just the vertices at or above that cut (per-thread histograms, parallel
    // compaction). The longest-prefix selection (R23) is unchanged: it stops inside the cut bucket.
    {
      const int nt = std::max(1, std::min(T, pool_size()));
      const int64_t nr = (int64_t)ranked.size();
      std::vector<uint64_t> vb((size_t)nr);
      auto bits = [](double x) {
        uint64_t b;
        std::memcpy(&b, &x, 8);
        return b;
      };
      std::vector<uint64_t> h1((size_t)nt * 4096, 0), h2((size_t)nt * 4096, 0);
      parallel_for(nt, nr, [&](int t, int64_t lo, int64_t hi) {
        uint64_t *h = &h1[(size_t)t * 4096];
        for (int64_t i = lo; i < hi; ++i) {
          vb[i] = (uint64_t)((S.view_len(ranked[i].second, VIEW_S) + 3u) & ~3u) * 4;
          if (ranked[i].first > 0) h[bits(ranked[i].first) >> 52] += vb[i];
        }
      });
      auto find_cut = [&](std::vector<uint64_t> &h, uint64_t before, uint32_t *cut, uint64_t *above) {
        uint64_t cum = before;
        for (int64_t b = 4095; b >= 0; --b) {
          uint64_t x = 0;
          for (int t = 0; t < nt; ++t) x += h[(size_t)t * 4096 + b];
          if (cum + x > ctx->budget) {
            *cut = (uint32_t)b;
            *above = cum;
            return true;
          }
          cum += x;
        }
        *cut = 0;
        *above = cum;
        return false;
      };
      uint32_t c1 = 0, c2 = 0;
      uint64_t above1 = 0, above2 = 0;
      const bool cut_found = find_cut(h1, 0, &c1, &above1);
      if (cut_found) {
        parallel_for(nt, nr, [&](int t, int64_t lo, int64_t hi) {
          uint64_t *h = &h2[(size_t)t * 4096];
          for (int64_t i = lo; i < hi; ++i)
            if (ranked[i].first > 0 && (bits(ranked[i].first) >> 52) == c1) h[(bits(ranked[i].first) >> 40) & 4095] += vb[i];
        });
        find_cut(h2, above1, &c2, &above2);
      }
      auto keep = [&](int64_t i) {
        if (!(ranked[i].first > 0)) return false;
        const uint64_t b = bits(ranked[i].first);
        const uint32_t k1 = (uint32_t)(b >> 52);
        return !cut_found || k1 > c1 || (k1 == c1 && ((b >> 40) & 4095) >= c2);
      };
      std::vector<int64_t> cnt((size_t)nt + 1, 0);
      parallel_for(nt, nr, [&](int t, int64_t lo, int64_t hi) {
        int64_t c = 0;
        for (int64_t i = lo; i < hi; ++i) c += keep(i);
        cnt[t + 1] = c;
      });
      for (int t = 0; t < nt; ++t) cnt[t + 1] += cnt[t];
      std::vector<std::pair<double, int32_t>> kept((size_t)cnt[nt]);
      parallel_for(nt, nr, [&](int t, int64_t lo, int64_t hi) {
        int64_t o = cnt[t];
        for (int64_t i = lo; i < hi; ++i)
          if (keep(i)) kept[o++] = ranked[i];
      });
      ranked.swap(kept);
    }
    parallel_sort(
        ranked,
        [](const std::pair<double, int32_t> &x, const std::pair<double, int32_t> &y) {
          return x.first > y.first || (x.first == y.first && x.second < y.second);
        },
        T);
    tr.mark("rank_sort");
    // list bytes of every ranked vertex (random accesses: in parallel), then the sequential prefix (R23)
    std::vector<uint64_t> rbytes(ranked.size());
    parallel_for(T, (int64_t)ranked.size(), [&](int, int64_t lo, int64_t hi) {
      for (int64_t i = lo; i < hi; ++i) rbytes[i] = (uint64_t)((S.view_len(ranked[i].second, VIEW_S) + 3u) & ~3u) * 4;
    });
    std::vector<uint64_t> bytes_of;
    for (size_t i = 0; i < ranked.size(); ++i) {
      if (!(ranked[i].first > 0)) break;
      if (used + rbytes[i] > ctx->budget) break;  // longest prefix that fits (R23)
      sel.push_back(ranked[i].second);
      bytes_of.push_back(rbytes[i]);
      used += rbytes[i];
    }
    // retained lists first, then the new ones
    for (int32_t v : ctx->prev_U) ctx->mark[v] = 2;
    std::vector<int64_t> old_off(sel.size(), -1);
    std::vector<uint64_t> src(sel.size(), 0);
    parallel_for(T, (int64_t)sel.size(), [&](int, int64_t lo, int64_t hi) {
      for (int64_t i = lo; i < hi; ++i) {
        const int32_t v = sel[i];
        if (ctx->cache_valid && ctx->mark[v] != 2 && S.uidx[v] < 0) {
          const uint32_t so = ctx->slot16[v];
          if (so) old_off[i] = 16 * (int64_t)(so - 1);
        }
        if (old_off[i] < 0) src[i] = (uint64_t)(uintptr_t)S.dev_ptr(S.view(v, VIEW_S).a);
      }
    });
    for (int32_t v : ctx->prev_U) ctx->mark[v] = 0;
    sel_off.assign(sel.size(), 0);
    uint64_t o = 0;
    for (size_t i = 0; i < sel.size(); ++i)
      if (old_off[i] >= 0) {
        sel_off[i] = o;
        gather.push_back((uint64_t)old_off[i]);
        gather.push_back(o);
        gather.push_back(bytes_of[i] / 16);
        o += bytes_of[i];
      }
    const uint64_t retained = o;
    // the newly selected lists are pulled by the GPU straight from the pinned host store (zero-copy bulk reads,
    // warp per list): the same bytes as the paper's packed DMA without a host-side packing copy
    for (size_t i = 0; i < sel.size(); ++i)
      if (old_off[i] < 0) {
        sel_off[i] = o;
        fresh.push_back(src[i]);
        fresh.push_back(o);
        fresh.push_back(bytes_of[i] / 16);
        o += bytes_of[i];
      }
    new_bytes = o - retained;
    tr.mark("layout");
  }
  tr.mark("stage_copy");
  st.cached_vertices = sel.size();
  st.cache_bytes = used;
  // descriptors to patch: previous cache / updated sets and the new ones
  std::vector<int32_t> dirty;
  static const std::vector<int32_t> kNone;
  {
    const std::vector<int32_t> *srcs[4] = {ctx->gpu_est ? &kNone : &ctx->prev_cached, &ctx->prev_U, &S.U,
                                           ctx->gpu_est ? &kNone : &sel};
    std::vector<int64_t> base(5, 0);
    for (int i = 0; i < 4; ++i) base[i + 1] = base[i] + (int64_t)srcs[i]->size();
    const int nt = std::max(1, std::min(T, pool_size()));
    std::vector<std::vector<int32_t>> part(nt);
    parallel_for(nt, base[4], [&](int tid, int64_t lo, int64_t hi) {
      for (int64_t g = lo; g < hi; ++g) {
        int l = 0;
        while (g >= base[l + 1]) ++l;
        const int32_t v = (*srcs[l])[g - base[l]];
        if (__atomic_exchange_n(&ctx->mark[v], (uint8_t)1, __ATOMIC_RELAXED) == 0) part[tid].push_back(v);
      }
    });
    for (auto &p : part) dirty.insert(dirty.end(), p.begin(), p.end());
    parallel_for(T, (int64_t)dirty.size(), [&](int, int64_t lo, int64_t hi) {
      for (int64_t i = lo; i < hi; ++i) ctx->mark[dirty[i]] = 0;
    });
  }
  if (ctx->sel_index.size() != (size_t)S.ncap) ctx->sel_index.assign(S.ncap, -1);
  for (size_t i = 0; i < sel.size(); ++i) ctx->sel_index[sel[i]] = (int32_t)i;
  if (!host_ensure(sl.h_pidx, sl.h_pidx_cap, dirty.size()) ||
      !host_ensure(sl.h_pval, sl.h_pval_cap, dirty.size()))
    return ctx->fail(GCSM_ENOMEM, "pinned staging");
  // GPU path: the stable lists S(x) of U travel with the batch (packed, 16-byte aligned, one DMA into this slot's
  // device buffer): every kernel of the batch reads them from HBM instead of re-reading the host overlays
  std::vector<uint64_t> ul_off;
  if (ctx->gpu_est) {
    const size_t nU0 = S.U.size();
    ul_off.assign(nU0 + 1, 0);
    for (size_t i = 0; i < nU0; ++i) ul_off[i + 1] = ul_off[i] + ((S.s_len[i] + 3u) & ~3u);
    sl.ulist_n = ul_off[nU0];
    if (!host_ensure(sl.h_ulist, sl.h_ulist_cap, sl.ulist_n) || !dev_ensure(sl.d_ulist, sl.d_ulist_cap, sl.ulist_n))
      return ctx->fail(GCSM_ENOMEM, "stable lists of U");
    parallel_for(T, (int64_t)nU0, [&](int, int64_t lo, int64_t hi) {
      for (int64_t i = lo; i < hi; ++i)
        if (S.s_len[i]) std::memcpy(sl.h_ulist + ul_off[i], S.s_ptr[i], 4 * (size_t)S.s_len[i]);
    });
  }
  parallel_for(T, (int64_t)dirty.size(), [&](int, int64_t lo, int64_t hi) {
    for (int64_t i = lo; i < hi; ++i) {
      const int32_t v = dirty[i];
      const int32_t ui = S.uidx[v];
      VDesc d;
      d.upd = ui >= 0 ? (uint32_t)ui + 1 : 0;
      d.len = ui >= 0 ? S.s_len[ui] : S.len[v];
      const int32_t si = ctx->sel_index[v];
      d.ptr = si >= 0 ? (const int32_t *)(ctx->d_cache + sel_off[si]) : S.dev_ptr(ui >= 0 ? S.s_ptr[ui] : S.lst[v]);
      if (ctx->gpu_est && ui >= 0) d.ptr = sl.d_ulist + ul_off[ui];
      sl.h_pidx[i] = v;
      sl.h_pval[i] = d;
    }
  });
  for (int32_t v : sel) ctx->sel_index[v] = -1;
  tr.mark("descriptors");
  // delta lists of U
  const size_t nU = S.U.size();
  const size_t nd = S.ins_val.size() + S.del_val.size();
  if (!host_ensure(sl.h_drec, sl.h_drec_cap, nU) || !host_ensure(sl.h_dlist, sl.h_dlist_cap, nd) ||
      !host_ensure(sl.h_units, sl.h_units_cap, (size_t)gnu))
    return ctx->fail(GCSM_ENOMEM, "pinned staging");
  for (size_t i = 0; i < nU; ++i)
    sl.h_drec[i] = DRec{S.ins_off[i], S.ins_off[i + 1] - S.ins_off[i], (uint32_t)S.ins_val.size() + S.del_off[i],
                          S.del_off[i + 1] - S.del_off[i]};
  std::memcpy(sl.h_dlist, S.ins_val.data(), S.ins_val.size() * 4);
  std::memcpy(sl.h_dlist + S.ins_val.size(), S.del_val.data(), S.del_val.size() * 4);
  for (int qi = 0; qi < nq; ++qi)
    if (!qunits[qi].empty())
      std::memcpy(sl.h_units + uoff[qi], qunits[qi].data(), sizeof(Unit) * qunits[qi].size());
  st.ms_pack = t3.ms();
  tr.mark("staging");

  cudaStream_t s = ctx->stream;
  // the cache step's stream: with overlap it runs beside the previous batch's matching (it writes only this slot's
  // descriptors, delta records, units and counters and the other cache buffer; the previous use of this slot was
  // batch t-2, already collected by gcsm_wait_batch)
  // (not with a query larger than overlap_kmax, default 8 since the late round-2 kernels; it was 5 while a 6-vertex query's level->=2 walks read zero-copy lists
  // and contend for the host link with the extension kernels they would run beside; GCSM_OVERLAP_KMAX
  // at create moves the limit)
  // Invariant of the overlapped step: k_sidx_update (in the cache step of t+1) rewrites the sampled index of batch
  // t's updated vertices while batch t's kernels may run; they never read it for those vertices, because the
  // descriptor of every x in U_t points into batch t's uploaded U buffer (is_hit() is true, the sampled index is
  // consulted only for zero-copy lists). A change that lets an updated vertex's descriptor point at host memory
  // must double-buffer soff per slot first.
  cudaStream_t cs = two_streams ? ctx->stream3 : s;
  if (!dev_ensure(ctx->d_pidx, ctx->pidx_cap, dirty.size()) || !dev_ensure(ctx->d_pval, ctx->pval_cap, dirty.size()) ||
      !dev_ensure(sl.d_drec, sl.drec_cap, nU) || !dev_ensure(sl.d_dlist, sl.dlist_cap, nd) ||
      !dev_ensure(sl.d_units, sl.units_cap, (size_t)gnu) || !dev_ensure(sl.d_useg, sl.useg_cap, (size_t)gnu))
    return ctx->fail(GCSM_ENOMEM, "device buffers");
  if (ctx->peers && ctx->batch_seq >= 2) {  // peers may still read this slot's descriptors and cache (batch t-2)
    std::lock_guard<std::mutex> lk(ctx->peers->mu);
    for (gcsm_ctx *p : ctx->peers->members)
      if (p != ctx) CK(cudaStreamWaitEvent(cs, p->slots[ctx->batch_seq & 1].ev_done, 0));
  }
  // fetch-once staging (k >= 5 extension kernels and walks): this slot's arena, allocated when first needed; the
  // batch's epoch and an empty arena, reset on the cache step's stream before its walks (the slot's previous user,
  // batch t-2, has completed: gcsm_wait_batch collected it)
  const bool staging = kmax >= 5 && !listing && ctx->opt.staging_bytes != 1 && !ctx->stage_failed;
  uint32_t stage_epoch = 0;
  gcsm_ctx::StageSlot &sg = ctx->stg[ctx->batch_seq & 1];
  if (staging) {
    if (!ctx->stg[0].arena) {
      size_t freeb = 0, totalb = 0;
      cudaMemGetInfo(&freeb, &totalb);
      size_t bytes = ctx->opt.staging_bytes ? ctx->opt.staging_bytes : std::min<size_t>(freeb / 4, (size_t)32 << 30);
      bytes = (bytes / 2) & ~(size_t)127;  // per slot
      bool ok = bytes >= 4096;
      for (auto &x : ctx->stg)
        ok = ok && cudaMalloc(&x.arena, bytes) == cudaSuccess &&
             cudaMalloc(&x.state, 8 * (size_t)S.ncap) == cudaSuccess && cudaMalloc(&x.bump, 8) == cudaSuccess;
      if (!ok) {
        cudaGetLastError();
        for (auto &x : ctx->stg) {
          for (void *p : {(void *)x.arena, (void *)x.state, (void *)x.bump})
            if (p) cudaFree(p);
          x = gcsm_ctx::StageSlot();
        }
        ctx->stage_failed = true;
      } else {
        for (auto &x : ctx->stg) {
          x.cap = bytes / 4;
          CK(cudaMemsetAsync(x.state, 0, 8 * (size_t)S.ncap, cs));
        }
      }
    }
    if (sg.arena) {
      stage_epoch = (uint32_t)(ctx->batch_seq % ((1u << 24) - 1)) + 1;  // 24 bits, never 0
      if (stage_epoch <= 2 && ctx->batch_seq > 1) CK(cudaMemsetAsync(sg.state, 0, 8 * (size_t)S.ncap, cs));
      CK(cudaMemsetAsync(sg.bump, 0, 8, cs));
    }
  }
  ctx->walk_stage_epoch = (stage_epoch && ctx->gpu_est) ? stage_epoch : 0;

  CK(cudaEventRecord(sl.ev_c0, cs));
  if (ctx->batch_seq > 0)  // this batch's descriptors start as the previous batch's (after its cache step)
    CK(cudaMemcpyAsync(sl.d_vdesc, ctx->slots[(ctx->batch_seq + 1) & 1].d_vdesc, sizeof(VDesc) * (size_t)S.n,
                       cudaMemcpyDeviceToDevice, cs));
  uint64_t launches = 0;
  if (ctx->gpu_est) {
    gcsm_status gs = enqueue_gpu_cache(ctx, sl, cs, dirty.size(), nU, nd, gnu, qeu, qitems, qf2cap, eu_maxB, D, qnu,
                                       qwalks, use_cache, &launches);
    if (gs != GCSM_OK) return gs;
    st.h2d_bytes = (sizeof(int64_t) + sizeof(VDesc)) * dirty.size() + sizeof(DRec) * nU + 4 * nd +
                   sizeof(Unit) * (size_t)gnu;
    for (const auto &eu : qeu) st.h2d_bytes += sizeof(EstUnit) * eu.size();
    st.h2d_bytes += 4 * sl.ulist_n;
  } else {
  const uint64_t retained_bytes = used - new_bytes;
  if (!gather.empty()) {  // HBM -> HBM copy of the retained lists from the previous buffer
    if (!host_ensure(sl.h_gather, sl.h_gather_cap, gather.size()) ||
        !dev_ensure(ctx->d_gather, ctx->gather_cap, gather.size()))
      return ctx->fail(GCSM_ENOMEM, "gather staging");
    std::memcpy(sl.h_gather, gather.data(), 8 * gather.size());
    CK(cudaMemcpyAsync(ctx->d_gather, sl.h_gather, 8 * gather.size(), cudaMemcpyHostToDevice, s));
    CK(launch_gather_lists(ctx->d_cache, ctx->d_cachebuf[ctx->cache_cur], ctx->d_gather, (int64_t)gather.size() / 3, s));
  }
  if (!fresh.empty()) {  // newly selected lists: GPU gather over PCIe from the mapped host store
    if (!host_ensure(sl.h_fresh, sl.h_fresh_cap, fresh.size()) ||
        !dev_ensure(ctx->d_fresh, ctx->fresh_cap, fresh.size()))
      return ctx->fail(GCSM_ENOMEM, "gather staging");
    std::memcpy(sl.h_fresh, fresh.data(), 8 * fresh.size());
    CK(cudaMemcpyAsync(ctx->d_fresh, sl.h_fresh, 8 * fresh.size(), cudaMemcpyHostToDevice, s));
    CK(launch_gather_lists(ctx->d_cache, nullptr, ctx->d_fresh, (int64_t)fresh.size() / 3, s));
  }
  (void)retained_bytes;
  CK(cudaMemcpyAsync(ctx->d_pidx, sl.h_pidx, sizeof(int64_t) * dirty.size(), cudaMemcpyHostToDevice, s));
  CK(cudaMemcpyAsync(ctx->d_pval, sl.h_pval, sizeof(VDesc) * dirty.size(), cudaMemcpyHostToDevice, s));
  CK(launch_patch_vdesc(sl.d_vdesc, ctx->d_pidx, ctx->d_pval, (int64_t)dirty.size(), s));
  launches += dirty.empty() ? 0 : 1;
  if (nU) CK(cudaMemcpyAsync(sl.d_drec, sl.h_drec, sizeof(DRec) * nU, cudaMemcpyHostToDevice, s));
  if (nd) CK(cudaMemcpyAsync(sl.d_dlist, sl.h_dlist, 4 * nd, cudaMemcpyHostToDevice, s));
  if (gnu) CK(cudaMemcpyAsync(sl.d_units, sl.h_units, sizeof(Unit) * (size_t)gnu, cudaMemcpyHostToDevice, s));
  CK(cudaEventRecord(sl.ev_c1, s));
  if (ctx->sp.n) CK(cudaEventRecord(ctx->ev_ipc[ctx->batch_seq & 1], s));
  st.h2d_bytes = new_bytes + 8 * gather.size() + 8 * fresh.size() + (sizeof(int64_t) + sizeof(VDesc)) * dirty.size() + sizeof(DRec) * nU +
                 4 * nd + sizeof(Unit) * (size_t)gnu;
  CK(cudaMemsetAsync(sl.d_cnt, 0, sizeof(unsigned long long) * CNT_N * (size_t)nq, s));
  }
  if (cs != s) CK(cudaStreamWaitEvent(s, sl.ev_c1, 0));  // the matching kernels read the cache step's output
  sl.cache_lo = ctx->d_cache;
  sl.cache_hi = ctx->d_cache ? ctx->d_cache + ctx->cache_cap : nullptr;
  // peer cache: rendezvous with the linked contexts at batch t (each has enqueued its cache step of t), then this
  // context's matching waits for theirs
  int npeer = 0;
  gcsm_ctx *peer_of[GCSM_MAX_PEERS] = {};
  if (ctx->peers) {
    PeerGroup &pg = *ctx->peers;
    std::unique_lock<std::mutex> lk(pg.mu);
    pg.enq[ctx->peer_idx] = ctx->batch_seq + 1;
    pg.cv.notify_all();
    pg.cv.wait(lk, [&] {
      for (uint64_t x : pg.enq)
        if (x < ctx->batch_seq + 1) return false;
      return true;
    });
    for (gcsm_ctx *p : pg.members)
      if (p != ctx && npeer < GCSM_MAX_PEERS) {
        CK(cudaStreamWaitEvent(s, p->slots[ctx->batch_seq & 1].ev_c1, 0));
        peer_of[npeer++] = p;
      }
  }

  // cross-process peers (node-shared store): publish which cache buffer this batch reads, meet every rank (each
  // has recorded its cache step of batch t), then this context's matching waits (device) for theirs. Slot reuse is
  // safe: a rank rewrites slot t & 1 (batch t+2) only after the store's entry barrier of t+2, which every rank
  // passes only after collecting batch t
  int snpeer = 0;
  const char *sp_lo[GCSM_MAX_PEERS] = {}, *sp_hi[GCSM_MAX_PEERS] = {}, *sp_map[GCSM_MAX_PEERS] = {};
  const VDesc *sp_vd[GCSM_MAX_PEERS] = {};
  if (ctx->sp.n && !ctx->peers) {
    const int slot = (int)(ctx->batch_seq & 1);
    PeerMail *me = reinterpret_cast<PeerMail *>(S.mailbox(S.store_rank()));
    me->cache_idx[slot] = !ctx->d_cache ? -1 : (ctx->d_cache == ctx->d_cachebuf[0] ? 0 : 1);
    std::atomic_thread_fence(std::memory_order_seq_cst);
    if (!S.barrier()) {
      ctx->poisoned = true;
      return ctx->fail(GCSM_ESTATE, S.shared_err);
    }
    for (int p = 0; p < ctx->sp.n && npeer + snpeer < GCSM_MAX_PEERS; ++p) {
      const PeerMail *pm = reinterpret_cast<const PeerMail *>(S.mailbox(ctx->sp.rank[p]));
      const int ci = pm->cache_idx[slot];
      if (ci < 0) continue;
      CK(cudaStreamWaitEvent(s, ctx->sp.ev[p][slot], 0));
      sp_vd[snpeer] = reinterpret_cast<const VDesc *>(ctx->sp.vdesc[p][slot]);
      sp_lo[snpeer] = reinterpret_cast<const char *>(ctx->sp.cache_va[p][ci]);
      sp_hi[snpeer] = sp_lo[snpeer] + ctx->sp.cache_cap[p];
      sp_map[snpeer] = ctx->sp.cache_map[p][ci];
      ++snpeer;
    }
  }

  // ---- (4) matching kernels (per query, in registration order, on the context stream) ---------------------
  const int dcap = (int)((D + 32 + 31) & ~uint64_t(31));
  // stacks + (list mode) last-level buffer + (k >= 5) hoisted set, filter set, level-3 iteration list
  const int nbuf = std::max(1, std::max(kmax - 4, 0) + (listing ? 1 : 0) + (kmax >= 5 ? 3 : 0));
  const size_t stride = (size_t)(nbuf + 3) * (size_t)dcap;  // stacks + pinned-x2 + 2 HBM staging buffers
  if (!dev_ensure(ctx->d_scratch, ctx->scratch_cap, stride * (size_t)ctx->warps_total))
    return ctx->fail(GCSM_ENOMEM, "scratch");
  // level-2 frontier chunks: per unit an upper bound on its candidates (unit indices local to the query)
  std::vector<std::vector<std::pair<int64_t, int64_t>>> qchunks((size_t)nq);
  std::vector<int64_t> qf2need((size_t)nq, 0);
  for (int qi = 0; qi < nq; ++qi) {
    int64_t &f2_need = qf2need[qi];
    const bool sym = !listing && ctx->qs[qi].qps.symmetry;
    const QueryPlan &QK = sym ? ctx->qs[qi].qps : ctx->qs[qi].qp;
    const std::vector<Unit> &units = qunits[qi];
    const int64_t qn = (int64_t)units.size();
    auto &chunks = qchunks[qi];
    if (QK.k >= 4) {
      int64_t start = 0, acc = 0;
      for (int64_t i = 0; i < qn; ++i) {
        const DevPlan &P = QK.plans[units[i].plan];
        const LevelPlan &L2 = P.lv[2];
        const int32_t f[2] = {units[i].a, units[i].b};
        int64_t b = INT64_MAX;
        for (int j = 0; j < L2.nb; ++j) b = std::min<int64_t>(b, S.view_len(f[L2.bpos[j]], L2.bview[j]));
        if (acc + b > kF2CapLimit && i > start) {
          chunks.push_back({start, i});
          f2_need = std::max(f2_need, acc);
          start = i;
          acc = 0;
        }
        acc += b;
      }
      chunks.push_back({start, qn});
      f2_need = std::max(f2_need, acc);
    } else {
      chunks.push_back({0, qn});
    }
  }
  for (int qi = 0; qi < nq; ++qi)
    if (ctx->qs[qi].qp.k >= 4 &&
        (!dev_ensure(ctx->d_f2q[qi], ctx->f2q_cap[qi], (size_t)std::max<int64_t>(2 * qf2need[qi], 2)) ||
         !dev_ensure(ctx->d_groupq[qi], ctx->groupq_cap[qi], (size_t)std::max<int64_t>(qf2need[qi], 1))))
      return ctx->fail(GCSM_ENOMEM, "frontier");
  // list mode buffers (one query)
  int32_t *d_tadd = nullptr, *d_trem = nullptr;
  if (listing) {
    const int k = ctx->qs[0].qp.k;
    const size_t need = (size_t)k * (add_cap + rem_cap);
    if (!dev_ensure(ctx->d_tup, ctx->tup_cap, std::max<size_t>(need, 1))) return ctx->fail(GCSM_ENOMEM, "tuples");
    d_tadd = ctx->d_tup;
    d_trem = ctx->d_tup + (size_t)k * add_cap;
  }
  MatchArgs A{};
  A.vdesc = sl.d_vdesc;
  A.lab = ctx->d_lab;
  A.drec = sl.d_drec;
  A.dlist = sl.d_dlist;

  A.scratch = ctx->d_scratch;
  A.scratch_end = ctx->d_scratch + stride * (size_t)ctx->warps_total;
  A.scratch_stride = (int64_t)stride;
  A.dcap = dcap;
  A.cache_lo = ctx->d_cache;
  A.cache_hi = ctx->d_cache ? ctx->d_cache + ctx->cache_cap : nullptr;
  A.ubuf_lo = ctx->gpu_est ? reinterpret_cast<const char *>(sl.d_ulist) : nullptr;
  A.ubuf_hi = ctx->gpu_est ? reinterpret_cast<const char *>(sl.d_ulist + sl.ulist_n) : nullptr;
  A.sidx = ctx->gpu_est && !std::getenv("GCSM_NO_SIDX") ? ctx->d_sidx : nullptr;
  A.soff = ctx->d_soff;
  A.tup_add = d_tadd;
  A.tup_add_cap = add_cap;
  A.tup_rem = d_trem;
  A.tup_rem_cap = rem_cap;
  A.listing = listing ? 1 : 0;
  if (stage_epoch) {
    A.stage_state = sg.state;
    A.stage_arena = sg.arena;
    A.stage_cap = sg.cap;
    A.stage_bump = sg.bump;
    A.stage_epoch = stage_epoch;
    A.stage_min = ctx->stage_min;
  }
  A.touched = ctx->bcomp ? ctx->d_touched_bc : nullptr;
  A.stage_policy = ctx->stage_policy;
  A.filter3 = std::getenv("GCSM_NO_FILTER3") ? 0 : 1;
  A.hoist = std::getenv("GCSM_NO_HOIST") ? 0 : 1;
  A.fsplit = std::getenv("GCSM_NO_FSPLIT") ? 0 : 1;
  A.merge2 = std::getenv("GCSM_MERGE2") ? 1 : 0;  // measured no faster on C3 / C4 (profiles/ab9_r02.txt)
  A.npeer = npeer + snpeer;
  for (int p = 0; p < npeer; ++p) {  // same process: the peer's addresses are ours
    const gcsm_ctx::Slot &ps = peer_of[p]->slots[ctx->batch_seq & 1];
    A.peer_vdesc[p] = ps.d_vdesc;
    A.peer_lo[p] = ps.cache_lo;
    A.peer_hi[p] = ps.cache_hi;
    A.peer_map[p] = ps.cache_lo;
  }
  for (int p = 0; p < snpeer; ++p) {  // other processes: their cache addresses are translated into our mapping
    A.peer_vdesc[npeer + p] = sp_vd[p];
    A.peer_lo[npeer + p] = sp_lo[p];
    A.peer_hi[npeer + p] = sp_hi[p];
    A.peer_map[npeer + p] = sp_map[p];
  }
  if (kmax >= 5 && !listing) {  // level-3 work sharing buffers (64M-int arena, 4M tasks)
    const size_t na = (size_t)64 << 20, nt = (size_t)4 << 20;
    const bool fresh_ready = ctx->d_task_ready == nullptr;
    if (!dev_ensure(ctx->d_arena, ctx->arena_cap, na) || !dev_ensure(ctx->d_tasks, ctx->tasks_cap, nt) ||
        !dev_ensure(ctx->d_task_ready, ctx->task_ready_cap, nt))
      return ctx->fail(GCSM_ENOMEM, "work-sharing buffers");
    if (fresh_ready) CK(cudaMemsetAsync(ctx->d_task_ready, 0, 4 * ctx->task_ready_cap, s));
  }
  while (sl.q.size() < (size_t)nq) {
    sl.q.emplace_back();
    CK(cudaEventCreate(&sl.q.back().ev_m0));
    CK(cudaEventCreate(&sl.q.back().ev_m1));
  }
  // per query and chunk: the kernel arguments (frontier buffers are per query, the unit segments per chunk)
  auto setup = [&](int qi, const std::pair<int64_t, int64_t> &ch) {
    const bool sym = !listing && ctx->qs[qi].qps.symmetry;
    const QueryPlan &QK = sym ? ctx->qs[qi].qps : ctx->qs[qi].qp;
    A.plans = sym ? ctx->qs[qi].d_splans : ctx->qs[qi].d_plans;
    A.n_plans = (int32_t)QK.plans.size();
    A.k = QK.k;
    A.cnt = sl.d_cnt + (size_t)qi * CNT_N;
    A.f2 = reinterpret_cast<int2 *>(ctx->d_f2q[qi]);
    A.f2_cap = qf2need[qi];
    A.units = sl.d_units + uoff[qi] + ch.first;
    A.n_units = ch.second - ch.first;
    A.useg = sl.d_useg + uoff[qi] + ch.first;
    A.group = nullptr;
    A.tasks = nullptr;
    if (QK.k >= 5 && !listing) {
      A.arena = ctx->d_arena;
      A.arena_cap = ctx->arena_cap;
      A.tasks = ctx->d_tasks;
      A.task_ready = ctx->d_task_ready;
      A.task_cap = (uint32_t)std::min<size_t>(ctx->tasks_cap, ctx->task_ready_cap);
    }
  };
  // level 2 + grouping of a chunk (events e0 / e1 around the level-2 kernel) on stream `st`
  auto level2 = [&](int qi, size_t ev0, cudaStream_t st) -> gcsm_status {
    auto &pq = sl.q[qi];
    unsigned long long *qcnt = sl.d_cnt + (size_t)qi * CNT_N;
    CK(cudaMemsetAsync(qcnt + CNT_F2, 0, sizeof(unsigned long long), st));
    CK(cudaMemsetAsync(qcnt + CNT_CURSOR0, 0, 2 * sizeof(unsigned long long), st));
    CK(cudaEventRecord(pq.kev[ev0], st));
    CK(launch_level2(A, ctx->grid, st));
    CK(cudaEventRecord(pq.kev[ev0 + 1], st));
    ++launches;
    if (A.k >= 4) {
      CK(launch_group_frontier(A, S.n, ctx->d_hist, ctx->d_bsum, ctx->d_groupq[qi], st));
      launches += 6;
    }
    return GCSM_OK;
  };
  for (int qi = 0; qi < nq; ++qi)
    while (sl.q[qi].kev.size() < 4 * std::max<size_t>(qchunks[qi].size(), 1)) {
      cudaEvent_t ev;
      CK(cudaEventCreate(&ev));
      sl.q[qi].kev.push_back(ev);
    }
  // GPU path: the first chunk's level-2 kernels read only the seeds' lists — the batch's uploaded U lists (R32) —
  // so they run on stream2 while the cache step runs on the main stream; the extensions wait for both
  const bool hoist = ctx->gpu_est && !ctx->bcomp;  // measurement mode: every kernel of a query on `s`, in order
  if (hoist) {
    CK(cudaStreamWaitEvent(ctx->stream2, sl.ev_up, 0));
    // the frontier buffers and grouping counters are shared with the previous batch's matching (stream order on
    // `stream` no longer implies it when the cache step runs beside it)
    if (ctx->batch_seq > 0) CK(cudaStreamWaitEvent(ctx->stream2, ctx->slots[(ctx->batch_seq + 1) & 1].ev_done, 0));
    for (int qi = 0; qi < nq; ++qi) {
      if (qchunks[qi].empty() || qchunks[qi][0].second <= qchunks[qi][0].first) continue;
      setup(qi, qchunks[qi][0]);
      gcsm_status g2 = level2(qi, 0, ctx->stream2);
      if (g2 != GCSM_OK) return g2;
    }
    CK(cudaEventRecord(sl.ev_l2, ctx->stream2));
    CK(cudaStreamWaitEvent(s, sl.ev_l2, 0));
  }
  for (int qi = 0; qi < nq; ++qi) {
    auto &pq = sl.q[qi];
    const bool sym = !listing && ctx->qs[qi].qps.symmetry;
    const QueryPlan &QK = sym ? ctx->qs[qi].qps : ctx->qs[qi].qp;
    const int k = QK.k;
    CK(cudaEventRecord(pq.ev_m0, s));
    if (ctx->bcomp) CK(cudaMemsetAsync(ctx->d_touched_bc, 0, 4 * (((size_t)S.n + 31) / 32), s));
    size_t nev = 0;
    for (size_t c = 0; c < qchunks[qi].size(); ++c) {
      const auto &ch = qchunks[qi][c];
      if (ch.second <= ch.first) continue;
      setup(qi, ch);
      if (!(hoist && c == 0)) {
        gcsm_status g2 = level2(qi, nev, s);
        if (g2 != GCSM_OK) return g2;
      }
      CK(cudaEventRecord(pq.kev[nev + 2], s));
      if (k >= 4) {
        A.group = ctx->d_groupq[qi];
        if (A.tasks) {
          if (++ctx->task_gen <= 0) ctx->task_gen = 1;  // ready flags hold the launch's generation, never 0
          A.task_gen = ctx->task_gen;
        }
        CK(launch_extend(A, ctx->ext_grid, s));
        ++launches;
      }
      CK(cudaEventRecord(pq.kev[nev + 3], s));
      nev += 4;
    }
    CK(cudaEventRecord(pq.ev_m1, s));
    if (ctx->bcomp) {
      CK(launch_bcomp(ctx->d_touched_bc, S.n, sl.d_vdesc, A.cache_lo, A.cache_hi, A.ubuf_lo, A.ubuf_hi,
                      sl.d_cnt + (size_t)qi * CNT_N + CNT_BCOMP, s));
      ++launches;
    }
    pq.nev = nev;
    pq.aut_mul = sym ? QK.automorphisms : 1;
  }
  // ---- (4b) count allreduce over NVLink (world > 1) -------------------------------------
  CK(cudaEventRecord(sl.ev_a0, s));
  if (ctx->comm) {  // ONE allreduce for every standing query: (added, removed) gathered into a packed buffer
    if (!dev_ensure(ctx->d_red, ctx->red_cap, 2 * (size_t)nq)) return ctx->fail(GCSM_ENOMEM, "allreduce buffer");
    const size_t pitch = sizeof(unsigned long long) * CNT_N, w16 = 2 * sizeof(unsigned long long);
    CK(cudaMemcpy2DAsync(ctx->d_red, w16, sl.d_cnt, pitch, w16, (size_t)nq, cudaMemcpyDeviceToDevice, s));
    if (ncclAllReduce(ctx->d_red, ctx->d_red, 2 * (size_t)nq, ncclUint64, ncclSum, ctx->comm, s) != ncclSuccess)
      return ctx->fail(GCSM_ENCCL, "ncclAllReduce failed");
    CK(cudaMemcpy2DAsync(sl.d_cnt, pitch, ctx->d_red, w16, w16, (size_t)nq, cudaMemcpyDeviceToDevice, s));
  }
  CK(cudaEventRecord(sl.ev_a1, s));
  CK(cudaMemcpyAsync(sl.h_cnt, sl.d_cnt, sizeof(unsigned long long) * CNT_N * (size_t)nq, cudaMemcpyDeviceToHost,
                     s));
  CK(cudaEventRecord(sl.ev_done, s));
  st.kernel_launches = launches;
  for (int qi = 0; qi < nq; ++qi) {  // shared steps' times and sizes, plus the query's own
    gcsm_stats &q = sl.q[qi].st;
    q = st;
    q.units = q.n1 = (uint64_t)qnu[qi];
    q.walks = qwalks[qi];
    q.ms_estimate = qms_est[qi];
  }
  sl.tup_add = tup_add;
  sl.tup_rem = tup_rem;
  sl.d_tadd = d_tadd;
  sl.d_trem = d_trem;
  sl.add_cap = add_cap;
  sl.rem_cap = rem_cap;
  tr.mark("enqueue");
  // ---- (5) reorganise the host lists. P:302 runs it after matching so the kernel reads consistent data: here
  // the merge writes fresh arrays and the ones the in-flight kernels may read are retired, not overwritten.
  Timer t5;
  if (!S.merge(sl.retired)) {
    if (S.shared()) {
      ctx->poisoned = true;
      return ctx->fail(GCSM_ESTATE, S.shared_err);
    }
    return ctx->fail(GCSM_ENOMEM, "pinned allocation for the merged lists failed");
  }
  tr.mark("merge");
  if (!ctx->gpu_est) {
    parallel_for(T, (int64_t)ctx->prev_cached.size(), [&](int, int64_t lo, int64_t hi) {
      for (int64_t i = lo; i < hi; ++i) ctx->slot16[ctx->prev_cached[i]] = 0;
    });
    parallel_for(T, (int64_t)sel.size(), [&](int, int64_t lo, int64_t hi) {
      for (int64_t i = lo; i < hi; ++i) ctx->slot16[sel[i]] = (uint32_t)(sel_off[i] / 16) + 1;
    });
    ctx->prev_cached.swap(sel);  // selection order (gcsm_get_cached sorts its copy)
  }
  if (ctx->budget > 0) {
    ctx->cache_cur = tgt;
    ctx->cache_valid = true;
  }
  ctx->prev_U = S.U;
  S.clear_batch();
  for (auto &pq : sl.q) pq.st.ms_merge = t5.ms();
  ++ctx->batch_seq;
  sl.inflight = true;
  sl.host_ms = total.ms();
  ctx->in_batch = false;
  ctx->err.clear();
  return GCSM_OK;
}


// Waits for the oldest in-flight batch and collects its counts and statistics.
static gcsm_status wait_impl(gcsm_ctx *ctx, uint64_t *added, uint64_t *removed) {
  if (!ctx) return GCSM_EINVAL;
  if (ctx->poisoned) return GCSM_ESTATE;
  if (ctx->waited >= ctx->batch_seq) return ctx->fail(GCSM_ESTATE, "no batch in flight");
  Timer tw;
  auto &sl = ctx->slots[ctx->waited & 1];
  CK(cudaEventSynchronize(sl.ev_done));
  const int nq = (int)ctx->qs.size();
  float ms_a = 0, ms_c = 0;
  cudaEventElapsedTime(&ms_a, sl.ev_a0, sl.ev_a1);
  cudaEventElapsedTime(&ms_c, sl.ev_c0, sl.ev_c1);
  bool trunc = false;
  for (int qi = 0; qi < nq; ++qi) {
    auto &pq = sl.q[qi];
    gcsm_stats st = pq.st;
    const unsigned long long *h = sl.h_cnt + (size_t)qi * CNT_N;
    if (h[CNT_OVERFLOW]) return ctx->fail(GCSM_EDEVICE, "internal: level-2 frontier overflow");
    if (ctx->gpu_est) {  // the GPU packer's selection (query 0's counter block; shared by all queries)
      const unsigned long long *h0 = sl.h_cnt;
      if (h0[CNT_CACHED + 2]) return ctx->fail(GCSM_EDEVICE, "internal: GPU estimator binomial table");
      st.cached_vertices = h0[CNT_CACHED];
      st.cache_bytes = h0[CNT_CACHED + 1];
    }
    st.ms_allreduce = ms_a;
    st.ms_copy = ms_c;
    for (size_t i = 0; i < pq.nev; i += 4) {  // per chunk: level 2 (e0 -> e1), extension (e2 -> e3)
      float a = 0, b = 0;
      cudaEventElapsedTime(&a, pq.kev[i], pq.kev[i + 1]);
      cudaEventElapsedTime(&b, pq.kev[i + 2], pq.kev[i + 3]);
      st.ms_level2 += a;
      st.ms_extend += b;
    }
    st.ms_match = st.ms_level2 + st.ms_extend;  // kernel time (the first level-2 launches overlap the cache step)
    st.added = h[CNT_ADDED] * pq.aut_mul;
    st.removed = h[CNT_REMOVED] * pq.aut_mul;
    st.hit_bytes_ext = h[CNT_ACC_EXT + 0];
    st.miss_bytes_ext = h[CNT_ACC_EXT + 1];
    st.delta_bytes_ext = h[CNT_ACC_EXT + 2];
    st.hit_bytes = h[CNT_ACC_L2 + 0] + st.hit_bytes_ext;
    st.miss_bytes = h[CNT_ACC_L2 + 1] + st.miss_bytes_ext;
    st.delta_bytes = h[CNT_ACC_L2 + 2] + st.delta_bytes_ext;
    st.host_copied_bytes = h[CNT_COPIED] + h[CNT_STAGE_FILL];  // warp staging copies + arena fills
    st.peer_bytes = h[CNT_PEER];
    st.walk_alg_bytes = h[CNT_WALG];
    st.walk_fill_bytes = sl.h_cnt[CNT_WFILL];  // the cache step's walks (all queries)
    st.walk_stage_lists = sl.h_cnt[CNT_WLISTS];
    st.ms_walks = 0;
    if (sl.walks_timed && (size_t)(2 * qi + 1) < sl.ev_walk.size() && ctx->qs[qi].qp.k > 2) {
      float mw = 0;
      if (cudaEventElapsedTime(&mw, sl.ev_walk[2 * qi], sl.ev_walk[2 * qi + 1]) == cudaSuccess) st.ms_walks = mw;
      cudaGetLastError();
    }
    st.stage_fill_bytes = h[CNT_STAGE_FILL];
    st.stage_lists = h[CNT_STAGE_LISTS];
    st.stage_hit_bytes = h[CNT_STAGE_HIT];
    st.bcomp_hit_bytes = h[CNT_BCOMP + 0];
    st.bcomp_miss_bytes = h[CNT_BCOMP + 1];
    st.bcomp_delta_bytes = h[CNT_BCOMP + 2];
    st.d2h_bytes = sizeof(unsigned long long) * CNT_N * (size_t)nq;
    st.frontier = h[CNT_F2];
    if (std::getenv("GCSM_TRACE"))
      std::fprintf(stderr, "[gcsm kern] q=%d frontier=%llu runs=%llu pins=%llu pin_gb=%.3f split_gb=%.3f copied_gb=%.3f "
                   "entries=%llu pruned=%llu l3=%llu l3kept=%llu l4=%llu last_drv=%llu\n",
                   qi, h[CNT_F2], h[CNT_DBG_RUNS], h[CNT_DBG_PINS], h[CNT_DBG_PINBYTES] / 1e9, h[CNT_DBG_SPLIT] / 1e9,
                   h[CNT_COPIED] / 1e9, h[CNT_X_ENTRIES], h[CNT_X_PRUNED], h[CNT_X_L3], h[CNT_X_L3F], h[CNT_X_L4], h[CNT_X_LAST]);
    if (std::getenv("GCSM_TRACE"))
      std::fprintf(stderr, "[gcsm ext-time] q=%d warps=%d ph1_mean_ms=%.2f ph1_max_ms=%.2f warp_max_ms=%.2f entry_max_ms=%.3f\n",
                   qi, ctx->warps_total, h[CNT_XT] / (double)ctx->warps_total / 1.965e6, h[CNT_XT + 1] / 1.965e6,
                   h[CNT_XT + 2] / 1.965e6, h[CNT_XT + 3] / 1.965e6);
    if (std::getenv("GCSM_TRACE"))
      std::fprintf(stderr, "[gcsm ext-phase] q=%d max_ms hoist=%.3f F=%.3f l3set=%.3f filter=%.3f rest=%.3f\n", qi,
                   h[CNT_XT + 4] / 1.965e6, h[CNT_XT + 5] / 1.965e6, h[CNT_XT + 6] / 1.965e6, h[CNT_XT + 7] / 1.965e6,
                   h[CNT_XT + 8] / 1.965e6);
    if (std::getenv("GCSM_TRACE"))
      std::fprintf(stderr, "[gcsm walks] q=%d roots=%llu lane_nodes=%llu dfs_descents=%llu steps=%llu walg_gb=%.3f\n", qi,
                   h[CNT_WDBG], h[CNT_WDBG + 1], h[CNT_WDBG + 2], h[CNT_WDBG + 3], h[CNT_WALG] / 1e9);
    if (qi == 0 && (sl.tup_add || sl.tup_rem)) {
      const int k = ctx->qs[0].qp.k;
      const uint64_t na = std::min<uint64_t>(h[CNT_TUP_ADD], sl.add_cap);
      const uint64_t nr = std::min<uint64_t>(h[CNT_TUP_REM], sl.rem_cap);
      if (na) CK(cudaMemcpy(sl.tup_add, sl.d_tadd, sizeof(int32_t) * k * na, cudaMemcpyDeviceToHost));
      if (nr) CK(cudaMemcpy(sl.tup_rem, sl.d_trem, sizeof(int32_t) * k * nr, cudaMemcpyDeviceToHost));
      st.d2h_bytes += sizeof(int32_t) * k * (na + nr);
      trunc = h[CNT_TUP_ADD] > sl.add_cap || h[CNT_TUP_REM] > sl.rem_cap;
      sl.tup_add = sl.tup_rem = nullptr;
    }
    st.ms_total = sl.host_ms + tw.ms();
    ctx->qs[qi].stats = st;
  }
  if (ctx->store.shared())  // other ranks' kernels may still read them: recycled at batch waited+2's first barrier
    ctx->pending_retired.emplace_back(ctx->waited, std::move(sl.retired)), sl.retired.clear();
  else
    ctx->store.recycle(sl.retired);  // arrays the batch's kernels could read are free again
  sl.inflight = false;
  ++ctx->waited;
  if (added) *added = ctx->qs[0].stats.added;
  if (removed) *removed = ctx->qs[0].stats.removed;
  if (trunc) return ctx->fail(GCSM_ETRUNC, "tuple buffer too small");
  ctx->err.clear();
  return GCSM_OK;
}

static gcsm_status apply_impl(gcsm_ctx *ctx, int64_t n_ins, const int32_t *ins, int64_t n_del, const int32_t *del,
                              int32_t *tup_add, uint64_t add_cap, int32_t *tup_rem, uint64_t rem_cap,
                              uint64_t *added, uint64_t *removed) {
  if (!ctx) return GCSM_EINVAL;
  while (ctx->waited < ctx->batch_seq) {  // drain batches submitted asynchronously
    gcsm_status w = wait_impl(ctx, nullptr, nullptr);
    if (w != GCSM_OK && w != GCSM_ETRUNC) return w;
  }
  gcsm_status e = submit_impl(ctx, n_ins, ins, n_del, del, tup_add, add_cap, tup_rem, rem_cap);
  if (e != GCSM_OK) return e;
  return wait_impl(ctx, added, removed);
}

extern "C" {

gcsm_status gcsm_apply_batch(gcsm_ctx *ctx, int64_t n_ins, const int32_t *ins, int64_t n_del, const int32_t *del,
                             uint64_t *added, uint64_t *removed) {
  return apply_impl(ctx, n_ins, ins, n_del, del, nullptr, 0, nullptr, 0, added, removed);
}

gcsm_status gcsm_apply_batch_list(gcsm_ctx *ctx, int64_t n_ins, const int32_t *ins, int64_t n_del, const int32_t *del,
                                  int32_t *added_tuples, uint64_t added_cap, int32_t *removed_tuples,
                                  uint64_t removed_cap, uint64_t *added, uint64_t *removed) {
  if (!added_tuples || !removed_tuples) return GCSM_EINVAL;
  return apply_impl(ctx, n_ins, ins, n_del, del, added_tuples, added_cap, removed_tuples, removed_cap, added,
                    removed);
}

gcsm_status gcsm_submit_batch(gcsm_ctx *ctx, int64_t n_ins, const int32_t *ins, int64_t n_del, const int32_t *del) {
  return submit_impl(ctx, n_ins, ins, n_del, del, nullptr, 0, nullptr, 0);
}

gcsm_status gcsm_wait_batch(gcsm_ctx *ctx, uint64_t *added, uint64_t *removed) {
  return wait_impl(ctx, added, removed);
}

gcsm_status gcsm_get_stats(const gcsm_ctx *ctx, gcsm_stats *out) {
  if (!ctx || !out) return GCSM_EINVAL;
  if (ctx->qs.empty()) {
    std::memset(out, 0, sizeof *out);
    return GCSM_OK;
  }
  *out = ctx->qs[0].stats;
  return GCSM_OK;
}

gcsm_status gcsm_get_query_stats(const gcsm_ctx *ctx, int32_t qid, gcsm_stats *out) {
  if (!ctx || !out || qid < 0 || (size_t)qid >= ctx->qs.size()) return GCSM_EINVAL;
  *out = ctx->qs[qid].stats;
  return GCSM_OK;
}

uint64_t gcsm_query_automorphisms(const gcsm_ctx *ctx) {
  return ctx && ctx->has_query ? ctx->qs[0].qp.automorphisms : 0;
}

gcsm_status gcsm_export_csr(const gcsm_ctx *ctx, int64_t *row_ptr, int32_t *col, uint64_t col_cap) {
  if (!ctx || !row_ptr) return GCSM_EINVAL;
  const HostStore &S = ctx->store;
  row_ptr[0] = 0;
  for (int32_t v = 0; v < S.n; ++v) row_ptr[v + 1] = row_ptr[v] + S.len[v];
  if (!col || col_cap < (uint64_t)row_ptr[S.n]) return GCSM_ETRUNC;
  for (int32_t v = 0; v < S.n; ++v)
    if (S.len[v]) std::memcpy(col + row_ptr[v], S.lst[v], (size_t)S.len[v] * 4);
  return GCSM_OK;
}

gcsm_status gcsm_get_estimates(const gcsm_ctx *ctx, int32_t *ids, uint64_t *levcnt, uint64_t cap, uint64_t *n_out) {
  if (!ctx || !n_out) return GCSM_EINVAL;
  if (ctx->gpu_est) {  // device-resident walk sums of the last batch (query 0): rows of the touched set, non-zero
    *n_out = 0;
    if (!ctx->est_valid || ctx->qs.empty() || ctx->qs[0].qp.k <= 2 || !ctx->d_levcnt[0]) return GCSM_OK;
    if (cudaStreamSynchronize(ctx->stream) != cudaSuccess || cudaStreamSynchronize(ctx->stream3) != cudaSuccess)
      return GCSM_EDEVICE;
    SelState st;
    if (cudaMemcpy(&st, ctx->d_sel, sizeof st, cudaMemcpyDeviceToHost) != cudaSuccess) return GCSM_EDEVICE;
    const int64_t nt = (int64_t)st.n_touched;
    std::vector<int32_t> tid((size_t)nt);
    std::vector<unsigned long long> rows((size_t)nt * 8);
    unsigned long long *d_rows = nullptr;
    if (nt) {
      if (cudaMalloc(&d_rows, 8 * 8 * (size_t)nt) != cudaSuccess) return GCSM_ENOMEM;
      cudaError_t e = launch_estimates_gather(ctx->d_tids, nt, ctx->d_levcnt[0], ctx->qs[0].qp.k - 2, d_rows,
                                              ctx->stream);
      if (e == cudaSuccess) e = cudaStreamSynchronize(ctx->stream);
      if (e == cudaSuccess) e = cudaStreamSynchronize(ctx->stream3);
      if (e == cudaSuccess) e = cudaMemcpy(rows.data(), d_rows, 8 * 8 * (size_t)nt, cudaMemcpyDeviceToHost);
      if (e == cudaSuccess) e = cudaMemcpy(tid.data(), ctx->d_tids, 4 * (size_t)nt, cudaMemcpyDeviceToHost);
      cudaFree(d_rows);
      if (e != cudaSuccess) return GCSM_EDEVICE;
    }
    uint64_t w = 0;
    for (int64_t i = 0; i < nt; ++i) {
      unsigned long long sum = 0;
      for (int l = 0; l < 8; ++l) sum |= rows[(size_t)i * 8 + l];
      if (!sum) continue;  // read only by other queries' walks
      if (w < cap) {
        if (ids) ids[w] = tid[i];
        if (levcnt) std::memcpy(levcnt + 8 * w, &rows[(size_t)i * 8], 64);
      }
      ++w;
    }
    *n_out = w;
    return w > cap ? GCSM_ETRUNC : GCSM_OK;
  }
  static const EstimatorOutput none;
  const EstimatorOutput &est = ctx->qs.empty() ? none : ctx->qs[0].est;
  const uint64_t n = est.ids.size();
  *n_out = n;
  const uint64_t w = std::min(n, cap);
  if (ids && w) std::memcpy(ids, est.ids.data(), 4 * w);
  if (levcnt && w) std::memcpy(levcnt, est.levcnt.data(), 8 * 8 * w);
  return n > cap ? GCSM_ETRUNC : GCSM_OK;
}

gcsm_status gcsm_get_cached(const gcsm_ctx *ctx, int32_t *ids, uint64_t cap, uint64_t *n_out) {
  if (!ctx || !n_out) return GCSM_EINVAL;
  if (ctx->gpu_est) {  // the GPU packer's last selection (ids ascending)
    *n_out = 0;
    if (!ctx->gpu_ready) return GCSM_OK;
    if (cudaStreamSynchronize(ctx->stream) != cudaSuccess || cudaStreamSynchronize(ctx->stream3) != cudaSuccess)
      return GCSM_EDEVICE;
    SelState st;
    if (cudaMemcpy(&st, ctx->d_sel, sizeof st, cudaMemcpyDeviceToHost) != cudaSuccess) return GCSM_EDEVICE;
    const uint64_t n = st.prev_sel, w = std::min<uint64_t>(n, cap);
    *n_out = n;
    if (ids && w && cudaMemcpy(ids, ctx->d_prev_sel, 4 * w, cudaMemcpyDeviceToHost) != cudaSuccess) return GCSM_EDEVICE;
    return n > cap ? GCSM_ETRUNC : GCSM_OK;
  }
  std::vector<int32_t> cached = ctx->prev_cached;
  std::sort(cached.begin(), cached.end());
  const uint64_t n = cached.size();
  *n_out = n;
  const uint64_t w = std::min(n, cap);
  if (ids && w) std::memcpy(ids, cached.data(), 4 * w);
  return n > cap ? GCSM_ETRUNC : GCSM_OK;
}

gcsm_status gcsm_plan_inspect(int32_t k, int32_t m, const int32_t *qedges, const int32_t *order, int32_t *out_seed,
                              int32_t *out_order, int32_t *out_nb, int32_t *out_bq, int32_t *out_view) {
  QueryPlan qp;
  if (!build_plan(k, m, qedges, nullptr, order, qp).empty()) return GCSM_EINVAL;
  for (int t = 0; t < m; ++t) {
    if (out_seed) {
      out_seed[2 * t] = qp.qe[t][0];
      out_seed[2 * t + 1] = qp.qe[t][1];
    }
    for (int kind = 0; kind < 2; ++kind) {
      const DevPlan &P = qp.plans[2 * t + kind];
      for (int p = 0; p < k; ++p) {
        if (kind == 0 && out_order) out_order[t * k + p] = P.order[p];
        const int nb = p >= 2 ? P.lv[p].nb : 0;
        if (kind == 0 && out_nb) out_nb[t * k + p] = nb;
        for (int b = 0; b < nb; ++b) {
          if (kind == 0 && out_bq) out_bq[(t * k + p) * 8 + b] = P.lv[p].bpos[b];
          if (out_view) out_view[((kind * m + t) * k + p) * 8 + b] = P.lv[p].bview[b];
        }
      }
    }
  }
  return GCSM_OK;
}

gcsm_status gcsm_query_restrictions(int32_t k, int32_t m, const int32_t *qedges, const int32_t *qlabels,
                                    const int32_t *order, int32_t *out_pairs, int32_t cap, int32_t *n_out,
                                    uint64_t *aut) {
  QueryPlan qp;
  if (!build_plan(k, m, qedges, qlabels, order, qp, true).empty()) return GCSM_EINVAL;
  const int32_t n = (int32_t)qp.restrictions.size();
  if (n_out) *n_out = n;
  if (aut) *aut = qp.automorphisms;
  for (int32_t i = 0; i < n && i < cap && out_pairs; ++i) {
    out_pairs[2 * i] = qp.restrictions[i].first;
    out_pairs[2 * i + 1] = qp.restrictions[i].second;
  }
  return n > cap ? GCSM_ETRUNC : GCSM_OK;
}

gcsm_status gcsm_binomial_samples(uint64_t key0, int64_t n, double p, int64_t count, int64_t *out) {
  if (count < 0 || n < 0 || !(p >= 0.0 && p <= 1.0) || (count > 0 && !out)) return GCSM_EINVAL;
  for (int64_t i = 0; i < count; ++i) out[i] = binomial(rng_chain(key0, (uint64_t)i), n, p);
  return GCSM_OK;
}

gcsm_status gcsm_shard(int64_t n_units, const uint64_t *cost, int32_t world, int32_t *out_rank) {
  if (n_units < 0 || world < 1 || (n_units && (!cost || !out_rank))) return GCSM_EINVAL;
  shard_lpt(n_units, cost, world, out_rank);
  return GCSM_OK;
}

}  // extern "C"
