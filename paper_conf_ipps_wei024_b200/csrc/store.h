// store.h — host dynamic-graph store (§V-A).
//
// The paper allocates one pinned, GPU-mapped array per vertex (cudaHostAlloc +
// cudaHostGetDevicePointer), appends insertions, marks deletions as -v
// and merges after matching. Here: one pinned mapped
// arena (a few large cudaHostAlloc chunks, 16-byte aligned lists, 2x capacity
// per list as P:270), and the batch is applied *out of place* as an overlay
// for the updated vertices U: stable list S(x) = N(x) \ del(x) (written to a
// pinned overlay area only when x has deletions), plus sorted ins(x) / del(x)
// — so every view (S, N = S ∪ del, N' = S ∪ ins) is a pair of sorted arrays
// (reading R13: no -v marks, vertex 0 is not ambiguous). Step ⑤ merges
// S(x) ∪ ins(x) into x's array (in place when the capacity allows, else a
// doubled relocation).
#pragma once
#include <cstdint>
#include <string>
#include <unordered_map>
#include <map>
#include <vector>

#include "estimator.h"
#include "internal.h"

namespace gcsm {

struct Chunk {
  char *host = nullptr;
  char *dev = nullptr;
  size_t size = 0, used = 0;
};

#define GCSM_MAX_STORE_RANKS 16
constexpr uint64_t kShmMailBytes = 4096;

// Node-shared store ("one shared shm arena cudaHostRegister'ed in each process"): one memfd mapping at
// the same virtual address in every local rank, so the list pointers in the shared per-vertex metadata are valid
// everywhere. Layout: this header (4 KiB), lst / len / cap / lab arrays (ncap each), two overlay areas (one per
// in-flight batch), the initial lists, then one growth region per rank (the merges of the vertices it owns,
// x % store_world == store_rank). See DESIGN.md §6.
struct ShmHeader {
  uint64_t magic, total_bytes, base_addr;
  int32_t n, ncap, world, labelled;
  int32_t leader_pid, fd;
  uint64_t off_lst, off_len, off_cap, off_lab, off_ovl[2], ovl_bytes, off_lists;
  uint64_t off_mail;  // per-rank mailboxes (kShmMailBytes each): the peer-cache IPC handles and per-batch state
  uint64_t reg_lo[GCSM_MAX_STORE_RANKS], reg_hi[GCSM_MAX_STORE_RANKS];
  std::atomic<uint64_t> reg_used[GCSM_MAX_STORE_RANKS];
  std::atomic<uint32_t> attached;
  std::atomic<uint32_t> failed;  // a rank poisoned its context: the others' barriers return false
  alignas(64) std::atomic<uint32_t> bar_count;
  alignas(64) std::atomic<uint32_t> bar_gen;
};

class HostStore {
 public:
  ~HostStore();
  // returns "" or an error message; *cuda_err set if the failure is a CUDA error
  // ncap >= n: vertex-id capacity (ids in [n, ncap) may join later, P:65 / P:273)
  std::string init(int32_t n, const int64_t *row_ptr, const int32_t *col, const int32_t *labels, int threads,
                   bool *cuda_err, int32_t ncap = 0);

  // node-shared store: store_rank 0 creates it (init with store_world > 1), the others attach to the handle
  std::string init_shared(int32_t n, const int64_t *row_ptr, const int32_t *col, const int32_t *labels, int threads,
                          bool *cuda_err, int store_world);
  std::string attach_shared(const char *handle, int32_t n, int threads, bool *cuda_err, int store_rank,
                            int store_world);
  std::string handle() const;  // "/proc/<pid>/fd/<fd>" of the leader's memfd ("" for a private store)
  bool shared() const { return shm_ != nullptr; }
  int store_rank() const { return srank_; }
  int store_world() const { return sworld_; }
  bool owned(int32_t x) const { return !shm_ || x % sworld_ == srank_; }
  void *mailbox(int rank) const {  // rank's kShmMailBytes-byte mailbox in the shared mapping (shared store only)
    return shm_ ? (char *)shm_ + shm_->off_mail + (uint64_t)rank * kShmMailBytes : nullptr;
  }
  // process-shared barrier of the store's ranks (no-op for a private store); false: timeout or a failed rank
  bool barrier();
  void poison_shared();
  std::string shared_err;  // why the last shared-store operation failed

  int32_t n = 0;     // current vertex count (ids [0, n))
  int32_t ncap = 0;  // capacity: every per-vertex array is sized ncap
  int threads = 1;
  int32_t **lst = nullptr;   // host address of each list (pinned, mapped); shared metadata with a shared store
  uint32_t *len = nullptr, *cap = nullptr;
  std::vector<uint16_t> lab;    // empty if unlabelled
  uint32_t maxdeg = 0;
  uint64_t edges2 = 0;          // Σ len

  const int32_t *dev_ptr(const int32_t *host) const;  // device-visible address of a pinned host address

  // ---- batch (steps ① / a0-a1) ----
  // Validates and normalises; on EINVAL returns the message and mutates nothing. Insertions may name ids in
  // [n, ncap) (new vertices): grow_n is then the vertex count the batch needs (grow() applies it).
  std::string normalize(int64_t n_ins, const int32_t *ins, int64_t n_del, const int32_t *del);
  int32_t grow_n = 0;
  // New vertices [n, new_n) ("allocate an array with an initial size of the average degree of the graph
  // for each new vertex"): empty lists of that capacity; false if the pinned allocation fails.
  bool grow(int32_t new_n);
  bool build_overlay(int slot, bool *cuda_err);  // S(x) for x ∈ U with deletions (per in-flight slot)
  HList view(int32_t v, int view) const;
  uint32_t view_len(int32_t v, int view) const;
  // step ⑤: base(x) <- S(x) ∪ ins(x) for x ∈ U, always into a *fresh* array (a recycled one of the same
  // capacity class, or a doubled one when full) so that a batch whose kernels are still reading
  // the old arrays (pipelined submit) is not disturbed; the old arrays are appended to `retired`.
  // With a shared store every rank computes the new lengths of all of U, then (after a barrier: every rank is done
  // reading G_t) merges only the vertices it owns, and a second barrier publishes G_{t+1}.
  bool merge(std::vector<std::pair<int32_t *, uint32_t>> &retired);  // false: pinned allocation failed
  void recycle(std::vector<std::pair<int32_t *, uint32_t>> &retired);  // once their batch has completed
  void clear_batch();

  // batch state
  std::vector<uint64_t> I, D;    // canonical keys (u << 32 | v), u < v, sorted
  uint64_t dropped = 0;
  std::vector<int32_t> U;        // updated vertices, ascending
  std::vector<int32_t> uidx;     // vertex -> index in U, or -1 (size n)
  std::vector<uint32_t> ins_off, del_off;  // size |U|+1, into ins_val / del_val
  std::vector<int32_t> ins_val, del_val;
  std::vector<const int32_t *> s_ptr;      // host address of S(x)
  std::vector<uint32_t> s_len;
  uint32_t maxdeg_new = 0;                 // max |N'(x)| over U
  std::vector<uint64_t> deg_hist;          // vertices per degree (exact max degree)

 private:
  std::vector<int32_t *> lst_v_;
  std::vector<uint32_t> len_v_, cap_v_;
  ShmHeader *shm_ = nullptr;
  size_t shm_size_ = 0;
  int srank_ = 0, sworld_ = 1;
  double bar_timeout_s_ = 600.0;
  std::string finish_shared_attach(bool *cuda_err);
  std::vector<Chunk> chunks_;
  Chunk overlay_[2];
  std::map<uint32_t, std::vector<int32_t *>> free_;  // recycled arrays by capacity
  // an array of >= capacity ints: a recycled one of up to 2x (capacity is raised to its size) or a fresh one
  int32_t *alloc_list(uint32_t &capacity, bool *cuda_err);
  bool new_chunk(size_t bytes, Chunk &c);
  size_t store_bytes_ = 0;  // pinned list capacity at init (growth quantum)
  bool has_edge(int32_t u, int32_t v) const;
};

}  // namespace gcsm
