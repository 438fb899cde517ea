// store.cpp — host dynamic-graph store (§V-A; see store.h).
#include "store.h"

#include <cuda_runtime.h>
#include <fcntl.h>
#include <linux/futex.h>
#include <sys/mman.h>
#include <sys/syscall.h>
#include <unistd.h>

#include <algorithm>
#include <atomic>
#include <cerrno>
#include <chrono>
#include <climits>
#include <cstdlib>
#include <cstring>
#include <thread>

namespace gcsm {

static inline uint32_t round4(uint64_t x) { return (uint32_t)((x + 3) & ~uint64_t(3)); }

HostStore::~HostStore() {
  if (shm_) {  // the mapping (and the leader's memfd) go away with the last process that maps it
    if (srank_ == 0) close(shm_->fd);
    cudaHostUnregister((void *)shm_);
    munmap((void *)shm_, shm_size_);
    return;
  }
  for (auto &c : chunks_)
    if (c.host) cudaFreeHost(c.host);
  for (auto &o : overlay_)
    if (o.host) cudaFreeHost(o.host);
}

bool HostStore::new_chunk(size_t bytes, Chunk &c) {
  void *h = nullptr;
  if (cudaHostAlloc(&h, bytes, cudaHostAllocMapped | cudaHostAllocPortable) != cudaSuccess) return false;
  void *d = nullptr;
  if (cudaHostGetDevicePointer(&d, h, 0) != cudaSuccess) {
    cudaFreeHost(h);
    return false;
  }
  c.host = (char *)h;
  c.dev = (char *)d;
  c.size = bytes;
  c.used = 0;
  return true;
}

const int32_t *HostStore::dev_ptr(const int32_t *host) const {
  if (!host) return nullptr;
  const char *p = (const char *)host;
  for (const auto &c : chunks_)
    if (p >= c.host && p < c.host + c.size) return (const int32_t *)(c.dev + (p - c.host));
  for (const auto &o : overlay_)
    if (o.host && p >= o.host && p < o.host + o.size) return (const int32_t *)(o.dev + (p - o.host));
  return nullptr;
}

int32_t *HostStore::alloc_list(uint32_t &capacity, bool *cuda_err) {
  // recycled array of the smallest capacity in [capacity, 2 capacity] (a retired list of a similar size)
  for (auto fit = free_.lower_bound(capacity); fit != free_.end() && fit->first <= 2ull * capacity; ++fit)
    if (!fit->second.empty()) {
      int32_t *p = fit->second.back();
      fit->second.pop_back();
      capacity = fit->first;  // the caller records the array's real capacity
      return p;
    }
  const size_t bytes = (size_t)capacity * 4;
  if (shm_) {  // this rank's growth region (only its owner allocates there; no new pinned chunks)
    const uint64_t used = shm_->reg_used[srank_].load(std::memory_order_relaxed);
    if (shm_->reg_lo[srank_] + used + bytes > shm_->reg_hi[srank_]) {
      shared_err = "the shared store's growth region of this rank is full";
      *cuda_err = true;
      return nullptr;
    }
    shm_->reg_used[srank_].store(used + bytes, std::memory_order_relaxed);
    return (int32_t *)((char *)shm_ + shm_->reg_lo[srank_] + used);
  }
  if (chunks_.empty() || chunks_.back().used + bytes > chunks_.back().size) {
    Chunk c;
    // grow by an eighth of the store at least: pinning memory (cudaHostAlloc) costs ~0.1-0.2 s per GB, so it
    // must be rare, not a per-batch stall
    size_t sz = std::max<size_t>(std::max<size_t>((size_t)256 << 20, 4 * bytes), store_bytes_ / 8);
    if (!new_chunk(sz, c)) {
      *cuda_err = true;
      return nullptr;
    }
    chunks_.push_back(c);
  }
  Chunk &c = chunks_.back();
  int32_t *p = (int32_t *)(c.host + c.used);
  c.used += bytes;  // capacities are multiples of 4 ints: 16-byte alignment kept
  return p;
}

static std::string validate_csr(int32_t n, const int64_t *rp, const int32_t *col, const int32_t *labels,
                                int threads) {
  if (n < 1) return "n must be >= 1";
  if (!rp || (rp[n] > 0 && !col)) return "row_ptr/col is NULL";
  if (rp[0] != 0) return "row_ptr[0] must be 0";
  for (int32_t v = 0; v < n; ++v)
    if (rp[v + 1] < rp[v]) return "row_ptr is not monotone";
  if (labels)
    for (int32_t v = 0; v < n; ++v)
      if (labels[v] < 0 || labels[v] > 65535) return "label out of [0, 65535]";
  // rows: in range, strictly ascending (no duplicates), no self loops; symmetric
  std::atomic<int> bad{0};
  parallel_for(threads, n, [&](int, int64_t lo, int64_t hi) {
    for (int64_t v = lo; v < hi && !bad.load(std::memory_order_relaxed); ++v) {
      for (int64_t e = rp[v]; e < rp[v + 1]; ++e) {
        const int32_t w = col[e];
        if (w < 0 || w >= n) { bad = 1; break; }
        if (w == v) { bad = 2; break; }
        if (e > rp[v] && col[e - 1] >= w) { bad = 3; break; }
        if (!std::binary_search(col + rp[w], col + rp[w + 1], (int32_t)v)) { bad = 4; break; }
      }
    }
  });
  switch (bad.load()) {
    case 1: return "column id out of range";
    case 2: return "self loop in the graph";
    case 3: return "row not strictly ascending (unsorted or duplicate)";
    case 4: return "graph is not symmetric";
    default: return "";
  }
}

std::string HostStore::init(int32_t n_, const int64_t *rp, const int32_t *col, const int32_t *labels, int threads_,
                            bool *cuda_err, int32_t ncap_) {
  *cuda_err = false;
  n = n_;
  ncap = std::max(n_, ncap_);
  threads = std::max(1, threads_);
  std::string e = validate_csr(n_, rp, col, labels, threads);
  if (!e.empty()) return e;
  lst_v_.assign(ncap, nullptr);
  len_v_.assign(ncap, 0);
  cap_v_.assign(ncap, 0);
  lst = lst_v_.data();
  len = len_v_.data();
  cap = cap_v_.data();
  uidx.assign(ncap, -1);
  if (labels) {
    lab.assign(ncap, 0);
    for (int32_t v = 0; v < n; ++v) lab[v] = (uint16_t)labels[v];
  }
  uint64_t total = 0;
  maxdeg = 0;
  for (int32_t v = 0; v < n; ++v) {
    const uint64_t d = (uint64_t)(rp[v + 1] - rp[v]);
    len[v] = (uint32_t)d;
    cap[v] = d ? round4(std::max<uint64_t>(4, 2 * d)) : 0;  // double the initial size
    total += cap[v];
    maxdeg = std::max<uint32_t>(maxdeg, (uint32_t)d);
  }
  edges2 = (uint64_t)rp[n];
  deg_hist.assign((size_t)maxdeg + 1, 0);
  for (int32_t v = 0; v < n; ++v) deg_hist[len[v]]++;
  Chunk c;
  store_bytes_ = total * 4;
  if (!new_chunk(total * 4 + std::max<size_t>((size_t)64 << 20, total / 2), c)) {  // slack: 1/8 of the store
    *cuda_err = true;
    return "cudaHostAlloc of the pinned store failed";
  }
  chunks_.push_back(c);
  size_t off = 0;
  for (int32_t v = 0; v < n; ++v) {
    if (cap[v]) {
      lst[v] = (int32_t *)(chunks_[0].host + off);
      off += (size_t)cap[v] * 4;
    }
  }
  chunks_[0].used = off;
  parallel_for(threads, n, [&](int, int64_t lo, int64_t hi) {
    for (int64_t v = lo; v < hi; ++v)
      if (len[v]) std::memcpy(lst[v], col + rp[v], (size_t)len[v] * 4);
  });
  return "";
}

// ---- node-shared store -------------------------------------------------------------------------------------

static constexpr uint64_t kShmMagic = 0x47435353544f5231ull;  // "GCSSTOR1"
static inline uint64_t align_up(uint64_t x, uint64_t a) { return (x + a - 1) / a * a; }

std::string HostStore::init_shared(int32_t n_, const int64_t *rp, const int32_t *col, const int32_t *labels,
                                   int threads_, bool *cuda_err, int store_world) {
  *cuda_err = false;
  if (store_world < 2 || store_world > GCSM_MAX_STORE_RANKS) return "store_world out of [2, 16]";
  n = ncap = n_;
  threads = std::max(1, threads_);
  std::string e = validate_csr(n_, rp, col, labels, threads);
  if (!e.empty()) return e;
  // sizes: the lists with 2x capacity, growth regions of 1/4 of that (split per rank), and two overlay
  // areas of 1/16 each (at least 256 MiB): S(x) of the updated vertices with deletions of one in-flight batch
  uint64_t total = 0;
  for (int32_t v = 0; v < n; ++v) {
    const uint64_t d = (uint64_t)(rp[v + 1] - rp[v]);
    total += d ? round4(std::max<uint64_t>(4, 2 * d)) : 0;
  }
  const uint64_t lists_b = total * 4, pg = 1 << 21;
  const uint64_t ovl_b = align_up(std::max<uint64_t>((uint64_t)256 << 20, lists_b / 16), pg);
  const uint64_t reg_b = align_up(std::max<uint64_t>((uint64_t)64 << 20, lists_b / 4 / (uint64_t)store_world), pg);
  ShmHeader hd{};
  uint64_t off = align_up(sizeof(ShmHeader), 4096);
  hd.off_lst = off; off = align_up(off + 8ull * n, 4096);
  hd.off_len = off; off = align_up(off + 4ull * n, 4096);
  hd.off_cap = off; off = align_up(off + 4ull * n, 4096);
  hd.off_lab = off; off = align_up(off + (labels ? 2ull * n : 0), 4096);
  hd.off_mail = off; off = align_up(off + kShmMailBytes * (uint64_t)store_world, pg);
  for (int sl = 0; sl < 2; ++sl) { hd.off_ovl[sl] = off; off += ovl_b; }
  hd.ovl_bytes = ovl_b;
  hd.off_lists = off; off = align_up(off + lists_b, pg);
  for (int r = 0; r < store_world; ++r) { hd.reg_lo[r] = off; off += reg_b; hd.reg_hi[r] = off; }
  const uint64_t bytes = off;
  const int fd = (int)syscall(SYS_memfd_create, "gcsm_store", 0u);
  if (fd < 0) return std::string("memfd_create: ") + std::strerror(errno);
  if (ftruncate(fd, (off_t)bytes) != 0) {
    close(fd);
    return std::string("ftruncate of the shared store: ") + std::strerror(errno);
  }
  // a high hint so that the other ranks can map the same range (MAP_FIXED_NOREPLACE there)
  void *base = mmap((void *)0x600000000000ull, bytes, PROT_READ | PROT_WRITE, MAP_SHARED, fd, 0);
  if (base == MAP_FAILED) {
    close(fd);
    return std::string("mmap of the shared store: ") + std::strerror(errno);
  }
  shm_ = (ShmHeader *)base;
  shm_size_ = bytes;
  new (shm_) ShmHeader();
  ShmHeader &h = *shm_;
  h.magic = 0;
  h.total_bytes = bytes;
  h.base_addr = (uint64_t)(uintptr_t)base;
  h.n = n;
  h.ncap = n;
  h.world = store_world;
  h.labelled = labels ? 1 : 0;
  h.leader_pid = (int32_t)getpid();
  h.fd = fd;  // kept open for the leader's lifetime: the other ranks open /proc/<pid>/fd/<fd>
  h.off_lst = hd.off_lst; h.off_len = hd.off_len; h.off_cap = hd.off_cap; h.off_lab = hd.off_lab;
  h.off_mail = hd.off_mail;
  h.off_ovl[0] = hd.off_ovl[0]; h.off_ovl[1] = hd.off_ovl[1]; h.ovl_bytes = ovl_b; h.off_lists = hd.off_lists;
  for (int r = 0; r < store_world; ++r) {
    h.reg_lo[r] = hd.reg_lo[r];
    h.reg_hi[r] = hd.reg_hi[r];
    h.reg_used[r].store(0);
  }
  h.attached.store(1);
  char *B = (char *)base;
  lst = (int32_t **)(B + h.off_lst);
  len = (uint32_t *)(B + h.off_len);
  cap = (uint32_t *)(B + h.off_cap);
  if (labels) {
    uint16_t *L = (uint16_t *)(B + h.off_lab);
    for (int32_t v = 0; v < n; ++v) L[v] = (uint16_t)labels[v];
  }
  size_t lo = 0;
  for (int32_t v = 0; v < n; ++v) {
    const uint64_t d = (uint64_t)(rp[v + 1] - rp[v]);
    len[v] = (uint32_t)d;
    cap[v] = d ? round4(std::max<uint64_t>(4, 2 * d)) : 0;
    lst[v] = cap[v] ? (int32_t *)(B + h.off_lists + lo) : nullptr;
    lo += (size_t)cap[v] * 4;
  }
  parallel_for(threads, n, [&](int, int64_t a, int64_t b) {
    for (int64_t v = a; v < b; ++v)
      if (len[v]) std::memcpy(lst[v], col + rp[v], (size_t)len[v] * 4);
  });
  store_bytes_ = lists_b;
  srank_ = 0;
  sworld_ = store_world;
  std::atomic_thread_fence(std::memory_order_seq_cst);
  h.magic = kShmMagic;
  return finish_shared_attach(cuda_err);
}

std::string HostStore::attach_shared(const char *handle, int32_t n_, int threads_, bool *cuda_err, int store_rank,
                                     int store_world) {
  *cuda_err = false;
  if (!handle || !*handle) return "empty shared-store handle";
  if (store_rank < 1 || store_rank >= store_world || store_world > GCSM_MAX_STORE_RANKS) return "bad store rank";
  threads = std::max(1, threads_);
  const int fd = open(handle, O_RDWR);
  if (fd < 0) return std::string("open ") + handle + ": " + std::strerror(errno);
  ShmHeader probe;
  if (pread(fd, &probe, sizeof probe, 0) != (ssize_t)sizeof probe || probe.magic != kShmMagic) {
    close(fd);
    return "not an initialised GCSM shared store";
  }
  if (probe.n != n_ || probe.world != store_world) {
    close(fd);
    return "shared store: n or store_world differs from the creating rank's";
  }
#ifndef MAP_FIXED_NOREPLACE
#define MAP_FIXED_NOREPLACE 0x100000
#endif
  void *want = (void *)(uintptr_t)probe.base_addr;
  void *base = mmap(want, probe.total_bytes, PROT_READ | PROT_WRITE, MAP_SHARED | MAP_FIXED_NOREPLACE, fd, 0);
  close(fd);
  if (base == MAP_FAILED || base != want) {
    if (base != MAP_FAILED) munmap(base, probe.total_bytes);
    return "shared store: its address range is taken in this process";
  }
  shm_ = (ShmHeader *)base;
  shm_size_ = probe.total_bytes;
  ShmHeader &h = *shm_;
  char *B = (char *)base;
  n = ncap = h.n;
  lst = (int32_t **)(B + h.off_lst);
  len = (uint32_t *)(B + h.off_len);
  cap = (uint32_t *)(B + h.off_cap);
  if (h.labelled) {
    lab.assign(ncap, 0);
    std::memcpy(lab.data(), B + h.off_lab, 2ull * n);
  }
  srank_ = store_rank;
  sworld_ = store_world;
  h.attached.fetch_add(1);
  return finish_shared_attach(cuda_err);
}

std::string HostStore::finish_shared_attach(bool *cuda_err) {
  ShmHeader &h = *shm_;
  if (const char *t = std::getenv("GCSM_SHM_TIMEOUT")) bar_timeout_s_ = std::atof(t);
  // every rank pins (and maps for its device) the whole range once
  if (cudaHostRegister((void *)shm_, shm_size_, cudaHostRegisterMapped | cudaHostRegisterPortable) != cudaSuccess) {
    cudaGetLastError();
    *cuda_err = true;
    return "cudaHostRegister of the shared store failed";
  }
  void *d = nullptr;
  if (cudaHostGetDevicePointer(&d, (void *)shm_, 0) != cudaSuccess) {
    *cuda_err = true;
    return "cudaHostGetDevicePointer of the shared store failed";
  }
  Chunk c;
  c.host = (char *)shm_;
  c.dev = (char *)d;
  c.size = c.used = shm_size_;
  chunks_.assign(1, c);  // dev_ptr() of every list and overlay
  for (int sl = 0; sl < 2; ++sl) {
    overlay_[sl].host = (char *)shm_ + h.off_ovl[sl];
    overlay_[sl].dev = (char *)d + h.off_ovl[sl];
    overlay_[sl].size = h.ovl_bytes;
  }
  uidx.assign(ncap, -1);
  maxdeg = 0;
  edges2 = 0;
  for (int32_t v = 0; v < n; ++v) {
    maxdeg = std::max(maxdeg, len[v]);
    edges2 += len[v];
  }
  deg_hist.assign((size_t)maxdeg + 1, 0);
  for (int32_t v = 0; v < n; ++v) deg_hist[len[v]]++;
  return "";
}

std::string HostStore::handle() const {
  if (!shm_) return "";
  return "/proc/" + std::to_string(shm_->leader_pid) + "/fd/" + std::to_string(shm_->fd);
}

void HostStore::poison_shared() {
  if (shm_) shm_->failed.store(1);
}

bool HostStore::barrier() {
  if (!shm_) return true;
  ShmHeader &h = *shm_;
  if (h.failed.load()) {
    shared_err = "another rank of the shared store failed";
    return false;
  }
  const uint32_t g = h.bar_gen.load(std::memory_order_acquire);
  if (h.bar_count.fetch_add(1, std::memory_order_acq_rel) + 1 == (uint32_t)sworld_) {
    h.bar_count.store(0, std::memory_order_relaxed);
    h.bar_gen.fetch_add(1, std::memory_order_release);
    syscall(SYS_futex, reinterpret_cast<uint32_t *>(&h.bar_gen), FUTEX_WAKE, INT_MAX, nullptr, nullptr, 0);
    return true;
  }
  const auto t0 = std::chrono::steady_clock::now();
  for (int spin = 0; h.bar_gen.load(std::memory_order_acquire) == g; ++spin) {
    if (spin < 4096) continue;
    timespec ts{0, 50 * 1000 * 1000};
    syscall(SYS_futex, reinterpret_cast<uint32_t *>(&h.bar_gen), FUTEX_WAIT, g, &ts, nullptr, 0);
    if (h.failed.load()) {
      shared_err = "another rank of the shared store failed";
      return false;
    }
    if (std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count() > bar_timeout_s_) {
      shared_err = "shared-store barrier timed out (a rank stopped calling the collective batch calls)";
      h.failed.store(1);
      return false;
    }
  }
  return true;
}

bool HostStore::grow(int32_t new_n) {
  if (new_n <= n) return true;
  if (new_n > ncap || shm_) return false;  // a shared store has no id growth (its capacity is n)
  const uint32_t avg = n > 0 ? (uint32_t)std::min<uint64_t>(edges2 / (uint64_t)n, 1u << 20) : 0;
  const uint32_t c0 = round4(std::max<uint32_t>(4, avg));
  bool err = false;
  for (int32_t v = n; v < new_n; ++v) {
    uint32_t c = c0;
    int32_t *p = alloc_list(c, &err);
    if (err) return false;
    lst[v] = p;
    cap[v] = c;
    len[v] = 0;
  }
  if (deg_hist.empty()) deg_hist.assign(1, 0);
  deg_hist[0] += (uint64_t)(new_n - n);
  n = new_n;
  return true;
}

bool HostStore::has_edge(int32_t u, int32_t v) const {
  if (len[u] > len[v]) std::swap(u, v);
  return std::binary_search(lst[u], lst[u] + len[u], v);
}

std::string HostStore::normalize(int64_t n_ins, const int32_t *ins, int64_t n_del, const int32_t *del) {
  if (n_ins < 0 || n_del < 0) return "negative batch size";
  if ((n_ins && !ins) || (n_del && !del)) return "batch pointer is NULL";
  auto keys = [&](int64_t m, const int32_t *e, std::vector<uint64_t> &out) -> std::string {
    out.resize(m);
    for (int64_t i = 0; i < m; ++i) {
      int32_t u = e[2 * i], v = e[2 * i + 1];
      if (u < 0 || v < 0 || u >= ncap || v >= ncap) return "vertex id out of range";
      if (e == del && (u >= n || v >= n)) return "a deleted edge names a vertex that does not exist (P:65)";
      if (u == v) return "self loop in batch";
      if (u > v) std::swap(u, v);
      out[i] = ((uint64_t)(uint32_t)u << 32) | (uint32_t)v;
    }
    std::sort(out.begin(), out.end());
    out.erase(std::unique(out.begin(), out.end()), out.end());
    return "";
  };
  std::vector<uint64_t> ki, kd;
  std::string err = keys(n_ins, ins, ki);
  if (!err.empty()) return err;
  err = keys(n_del, del, kd);
  if (!err.empty()) return err;
  for (size_t i = 0, j = 0; i < ki.size() && j < kd.size();) {
    if (ki[i] == kd[j]) return "edge both inserted and deleted";
    if (ki[i] < kd[j]) ++i;
    else ++j;
  }
  // --- no mutation before this point ---
  grow_n = n;
  for (uint64_t key : ki) grow_n = std::max<int32_t>(grow_n, (int32_t)(key & 0xffffffffu) + 1);
  I.clear();
  D.clear();
  dropped = 0;
  // existence checks: random probes into the host lists, in parallel
  std::vector<uint8_t> ei(ki.size()), ed(kd.size());
  parallel_for(threads, (int64_t)(ki.size() + kd.size()), [&](int, int64_t lo, int64_t hi) {
    for (int64_t i = lo; i < hi; ++i) {
      const uint64_t key = i < (int64_t)ki.size() ? ki[i] : kd[i - ki.size()];
      const uint8_t h = has_edge((int32_t)(key >> 32), (int32_t)(key & 0xffffffffu));
      if (i < (int64_t)ki.size()) ei[i] = h;
      else ed[i - ki.size()] = h;
    }
  });
  for (size_t i = 0; i < ki.size(); ++i) {
    if (ei[i]) ++dropped;
    else I.push_back(ki[i]);
  }
  for (size_t i = 0; i < kd.size(); ++i) {
    if (ed[i]) D.push_back(kd[i]);
    else ++dropped;
  }
  // directed pairs grouped by source
  auto directed = [](const std::vector<uint64_t> &E) {
    std::vector<uint64_t> d;
    d.reserve(2 * E.size());
    for (uint64_t key : E) {
      d.push_back(key);
      d.push_back(((key & 0xffffffffu) << 32) | (key >> 32));
    }
    std::sort(d.begin(), d.end());
    return d;
  };
  const std::vector<uint64_t> di = directed(I), dd = directed(D);
  U.clear();
  for (uint64_t x : di) U.push_back((int32_t)(x >> 32));
  for (uint64_t x : dd) U.push_back((int32_t)(x >> 32));
  std::sort(U.begin(), U.end());
  U.erase(std::unique(U.begin(), U.end()), U.end());
  for (size_t i = 0; i < U.size(); ++i) uidx[U[i]] = (int32_t)i;
  ins_off.assign(U.size() + 1, 0);
  del_off.assign(U.size() + 1, 0);
  ins_val.resize(di.size());
  del_val.resize(dd.size());
  for (size_t i = 0; i < di.size(); ++i) {
    ins_off[uidx[(int32_t)(di[i] >> 32)] + 1]++;
    ins_val[i] = (int32_t)(di[i] & 0xffffffffu);
  }
  for (size_t i = 0; i < dd.size(); ++i) {
    del_off[uidx[(int32_t)(dd[i] >> 32)] + 1]++;
    del_val[i] = (int32_t)(dd[i] & 0xffffffffu);
  }
  for (size_t i = 0; i < U.size(); ++i) {
    ins_off[i + 1] += ins_off[i];
    del_off[i + 1] += del_off[i];
  }
  return "";
}

bool HostStore::build_overlay(int slot, bool *cuda_err) {
  *cuda_err = false;
  Chunk &overlay_ = this->overlay_[slot & 1];
  const size_t nu = U.size();
  s_ptr.assign(nu, nullptr);
  s_len.assign(nu, 0);
  std::vector<size_t> off(nu + 1, 0);
  for (size_t i = 0; i < nu; ++i) {
    const bool has_del = del_off[i + 1] > del_off[i];
    off[i + 1] = off[i] + (has_del ? round4(len[U[i]]) : 0);
  }
  const size_t bytes = off[nu] * 4 + 64;
  if (shm_ && overlay_.size < bytes) {
    shared_err = "the batch's stable lists exceed the shared store's overlay area";
    return false;
  }
  if (overlay_.size < bytes) {
    if (overlay_.host) cudaFreeHost(overlay_.host);
    overlay_ = Chunk();
    if (!new_chunk(std::max<size_t>(bytes * 2, (size_t)16 << 20), overlay_)) {
      *cuda_err = true;
      return false;
    }
  }
  maxdeg_new = 0;
  std::vector<uint32_t> newdeg(nu);
  parallel_for(threads, (int64_t)nu, [&](int, int64_t lo, int64_t hi) {
    for (int64_t i = lo; i < hi; ++i) {
      const int32_t x = U[i];
      const int32_t *dl = del_val.data() + del_off[i];
      const uint32_t nd = del_off[i + 1] - del_off[i];
      if (nd == 0) {
        s_ptr[i] = lst[x];
        s_len[i] = len[x];
      } else if (!owned(x)) {  // shared store: x's owner writes S(x); del(x) ⊆ N(x) after normalisation
        s_ptr[i] = (int32_t *)(overlay_.host) + off[i];
        s_len[i] = len[x] - nd;
      } else {
        int32_t *out = (int32_t *)(overlay_.host) + off[i];
        const int32_t *e = std::set_difference(lst[x], lst[x] + len[x], dl, dl + nd, out);
        s_ptr[i] = out;
        s_len[i] = (uint32_t)(e - out);
      }
      newdeg[i] = s_len[i] + (ins_off[i + 1] - ins_off[i]);
    }
  });
  for (size_t i = 0; i < nu; ++i) maxdeg_new = std::max(maxdeg_new, newdeg[i]);
  return barrier();  // shared store: every owner's S(x) is written before any rank reads it
}

HList HostStore::view(int32_t v, int vw) const {
  const int32_t i = uidx[v];
  if (i < 0) return HList{lst[v], len[v], nullptr, 0};
  HList h{s_ptr[i], s_len[i], nullptr, 0};
  if (vw == VIEW_NEW) {
    h.b = ins_val.data() + ins_off[i];
    h.nb = ins_off[i + 1] - ins_off[i];
  } else if (vw == VIEW_OLD) {
    h.b = del_val.data() + del_off[i];
    h.nb = del_off[i + 1] - del_off[i];
  }
  return h;
}

uint32_t HostStore::view_len(int32_t v, int vw) const {
  const int32_t i = uidx[v];
  if (i < 0) return len[v];
  if (vw == VIEW_NEW) return s_len[i] + ins_off[i + 1] - ins_off[i];
  if (vw == VIEW_OLD) return s_len[i] + del_off[i + 1] - del_off[i];
  return s_len[i];
}

bool HostStore::merge(std::vector<std::pair<int32_t *, uint32_t>> &retired) {
  const size_t nu = U.size();
  std::vector<int32_t *> target(nu, nullptr);
  std::vector<uint32_t> newlen(nu), newcap(nu), oldlen(nu);
  for (size_t i = 0; i < nu; ++i) {
    const int32_t x = U[i];
    oldlen[i] = len[x];
    newlen[i] = s_len[i] + (ins_off[i + 1] - ins_off[i]);
    newcap[i] = cap[x];
    if (newlen[i] > cap[x]) newcap[i] = round4(std::max<uint64_t>(4, 2ull * newlen[i]));  // double
  }
  // shared store: every rank has read G_t's metadata for this batch before any owner rewrites it
  if (!barrier()) return false;
  bool err = false;
  for (size_t i = 0; i < nu; ++i) {
    if (!owned(U[i])) continue;
    target[i] = newcap[i] ? alloc_list(newcap[i], &err) : nullptr;  // may raise newcap[i] (recycled array)
    if (err) {  // give back what this merge took; the store is unchanged
      for (size_t j = 0; j < i; ++j)
        if (target[j]) free_[newcap[j]].push_back(target[j]);
      poison_shared();
      return false;
    }
  }
  parallel_for(threads, (int64_t)nu, [&](int, int64_t lo, int64_t hi) {
    for (int64_t i = lo; i < hi; ++i) {
      const int32_t *in = ins_val.data() + ins_off[i];
      const uint32_t ni = ins_off[i + 1] - ins_off[i];
      if (target[i]) std::merge(s_ptr[i], s_ptr[i] + s_len[i], in, in + ni, target[i]);
    }
  });
  for (size_t i = 0; i < nu; ++i) {
    const int32_t x = U[i];
    deg_hist[oldlen[i]]--;
    if (newlen[i] >= deg_hist.size()) deg_hist.resize((size_t)newlen[i] + 1, 0);
    deg_hist[newlen[i]]++;
    edges2 += newlen[i];
    edges2 -= oldlen[i];
    if (!owned(x)) continue;
    if (lst[x]) retired.push_back({lst[x], cap[x]});
    len[x] = newlen[i];
    cap[x] = newcap[i];
    lst[x] = target[i];
  }
  maxdeg = (uint32_t)deg_hist.size() - 1;
  while (maxdeg > 0 && deg_hist[maxdeg] == 0) --maxdeg;
  return barrier();  // shared store: G_{t+1} is published to every rank
}

void HostStore::recycle(std::vector<std::pair<int32_t *, uint32_t>> &retired) {
  for (auto &r : retired) free_[r.second].push_back(r.first);
  retired.clear();
}

void HostStore::clear_batch() {
  for (int32_t x : U) uidx[x] = -1;
  U.clear();
  I.clear();
  D.clear();
}

}  // namespace gcsm
