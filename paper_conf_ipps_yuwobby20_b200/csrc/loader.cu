// loader.cu — host side of libgdroid.so: the C ABI of include/gdroid.h.
//
// (a1) validates each app's ICFG (V1-V6 of DESIGN.md §3), resolves every operand to a row of
// its node's fact block, lays out the fact store (node-major MAT blocks),
// builds the cross-module projection tables and uploads everything with one pinned staging
// buffer (the paper's dual-buffered copy, Alg. 2 l.2, is recast as the corpus driver's
// double-buffered per-batch H2D).  (a2)-(a7) are enqueued by gdroid_build_idfg.
#include <algorithm>
#include <cstdlib>
#include <chrono>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <atomic>
#include <condition_variable>
#include <functional>
#include <map>
#include <memory>
#include <new>
#include <mutex>
#include <thread>
#include <unordered_map>
#include <string>
#include <vector>

#include "internal.cuh"

using namespace gd;

namespace {

#ifndef GD_HYBRID
#define GD_HYBRID 1          // large narrow batches alternate the 3- and 4-CTA/SM instantiations
#endif
constexpr uint32_t HYB_SWITCHES = 8;
#ifndef GD_HYB_HI
#define GD_HYB_HI 16         // heavy round: >= GD_HYB_HI/4 waves of items (3-CTA grid)
#endif
#ifndef GD_HYB_LO
#define GD_HYB_LO 4          // light round: < GD_HYB_LO/4 waves
#endif

thread_local std::string g_err;

// GDROID_TIMING=1: print host-side phase times of gdroid_load_* to stderr
struct PhaseTimer {
  bool on;
  std::chrono::steady_clock::time_point t;
  PhaseTimer() : on(getenv("GDROID_TIMING") != nullptr), t(std::chrono::steady_clock::now()) {}
  void mark(const char* what) {
    if (!on) return;
    auto now = std::chrono::steady_clock::now();
    fprintf(stderr, "[gdroid] %-28s %8.2f ms\n", what, std::chrono::duration<double, std::milli>(now - t).count());
    t = now;
  }
};
thread_local PhaseTimer* g_pt = nullptr;
#define PHASE(x) do { if (g_pt) g_pt->mark(x); } while (0)

gdroid_status set_err(gdroid_status st, const char* fmt, ...) {
  char buf[600];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  g_err = buf;
  return st;
}

#define CU(call)                                                                          \
  do {                                                                                    \
    cudaError_t _e = (call);                                                              \
    if (_e != cudaSuccess)                                                                \
      return set_err(_e == cudaErrorMemoryAllocation ? GDROID_E_OOM : GDROID_E_CUDA,      \
                     "%s failed: %s", #call, cudaGetErrorString(_e));                     \
  } while (0)

template <class T>
int64_t bsearch_idx(const T* a, uint64_t n, T key) {
  const T* p = std::lower_bound(a, a + n, key);
  return (p != a + n && *p == key) ? (int64_t)(p - a) : -1;
}

uint32_t cls_of(uint8_t k) {
  switch (k) {
    case GK_COPY: case GK_SLOAD: case GK_SSTORE: case GK_RETV: return C_SINGLE;      // (ii)
    case GK_FLOAD: case GK_FSTORE: case GK_ALOAD: case GK_ASTORE: return C_DOUBLE;   // (iii)
    case GK_CALL: return C_CALL;
    case GK_EXIT: return C_EXIT;
    default: return C_ONETIME;                                                      // (i)
  }
}

// Allocator whose resize() leaves new elements uninitialised (large tables are filled in parallel).
template <class T>
struct NoInit : std::allocator<T> {
  template <class U> struct rebind { using other = NoInit<U>; };
  template <class U, class... A> void construct(U* p, A&&... a) {
    if constexpr (sizeof...(A) == 0) ::new ((void*)p) U; else ::new ((void*)p) U(std::forward<A>(a)...);
  }
};

// Host images of every device table of a batch.
struct HostImage {
  // per-node tables are written straight into the pinned staging buffer (region A) with
  // app-local indices; k_rebase adds the app's bases on the device
  NodeRec* o_nodes = nullptr;
  uint32_t* o_nodemeth = nullptr;
  uint32_t* o_rowptr = nullptr;                // [n + 1] of this app's node n
  uint32_t* o_argptr = nullptr;
  uint64_t n_nodes = 0;
  std::vector<MethRec> meths;
  std::vector<ModRec> mods;
  // edges: the device builds the Edge / InlEdge records (k_edges) from the descriptor's col and
  // edge_kind plus the projection-table offset of each CALL/RET edge computed here
  const gdroid_icfg_desc* desc = nullptr;
  uint64_t n_edges = 0;
  std::vector<uint32_t, NoInit<uint32_t>> xo; // [E] app-local xmap offset | NO_XMAP (all written)
  std::vector<int32_t> args;
  std::vector<uint32_t> col_gid, col_hbase;
  std::vector<int32_t> col_type;
  std::vector<uint32_t> grow_gid;
  std::vector<int32_t> grow_col, grow_field;
  std::vector<uint32_t> tf_ptr{0}, tf;
  std::vector<int32_t, NoInit<int32_t>> xmap;  // projection tables: colmap then rowmap (filled in parallel)
  std::vector<int32_t> frow;                   // per (module, field): column -> global heap row | -1
  std::vector<uint32_t> app_node_base;
  std::vector<uint32_t> entries;
  uint64_t fact_words = 0;
  uint32_t cls_count[NCLS] = {0, 0, 0, 0, 0};
  // per-load temporaries, kept so their pages are touched once per process (first-touch faults
  // cost more than the table build itself in this environment)
  std::vector<uint64_t> t_heap_base, t_local_base, t_msize;
  std::vector<uint64_t, NoInit<uint64_t>> t_foff;             // every entry written by the size pass
  std::vector<uint8_t> t_kmark, t_pmark;
  std::vector<uint32_t> t_kidx, t_pidx;
};

// Per-module host-side lookup info of the app being loaded.
struct ModInfo {
  const uint32_t* insts; uint64_t n_insts;
  const uint32_t* stats; uint64_t n_stats;
  uint32_t gmod;   // global module index
};

// Persistent worker pool for the host-side table build (spawning threads per parallel loop
// costs more than the loops themselves on small apps).  Nested loops are allowed: a
// parallel_for called from inside a task publishes its own job and its caller works on it (and
// on any other open job) until it completes, so apps and node ranges inside apps share the
// pool.
class Pool {
 public:
  struct Job {
    const std::function<void(uint32_t)>* f = nullptr;
    uint32_t n = 0;
    std::atomic<uint32_t> next{0}, done{0}, refs{0};
  };
  static Pool& get() {
    static Pool p;
    return p;
  }
  uint32_t size() const { return (uint32_t)workers_.size() + 1; }
  void run(uint32_t n, const std::function<void(uint32_t)>& f) {
    Job j;
    j.f = &f; j.n = n;
    {
      std::lock_guard<std::mutex> lk(mu_);
      jobs_.push_back(&j);
    }
    cv_.notify_all();
    for (uint32_t k; (k = j.next.fetch_add(1)) < n;) { f(k); j.done.fetch_add(1); }
    while (j.done.load() < n || j.refs.load() != 0)
      if (!help_one()) std::this_thread::yield();
    std::lock_guard<std::mutex> lk(mu_);
    for (size_t i = 0; i < jobs_.size(); ++i)
      if (jobs_[i] == &j) { jobs_.erase(jobs_.begin() + i); break; }
  }

 private:
  Pool() {
    // GDROID_HOST_THREADS caps the pool (several ranks per host share its cores)
    uint32_t T = std::max(1u, std::thread::hardware_concurrency());
    if (const char* e = getenv("GDROID_HOST_THREADS")) {
      const long v = strtol(e, nullptr, 10);
      if (v > 0) T = std::min<uint32_t>(T, (uint32_t)v);
    }
    for (uint32_t t = 1; t < T; ++t) workers_.emplace_back([this] { loop(); });
  }
  ~Pool() {
    { std::lock_guard<std::mutex> lk(mu_); stop_ = true; }
    cv_.notify_all();
    for (auto& w : workers_) w.join();
  }
  // Claim and run one index of an open job; false if there is none.  refs keeps the job (on its
  // caller's stack) alive while a helper holds it.
  bool help_one() {
    Job* j = nullptr;
    {
      std::lock_guard<std::mutex> lk(mu_);
      for (size_t i = 0; i < jobs_.size(); ++i)
        if (jobs_[i]->next.load() < jobs_[i]->n) { j = jobs_[i]; break; }
      if (!j) return false;
      j->refs.fetch_add(1);
    }
    const uint32_t k = j->next.fetch_add(1);
    if (k < j->n) { (*j->f)(k); j->done.fetch_add(1); }
    j->refs.fetch_sub(1);
    return true;
  }
  void loop() {
    for (;;) {
      if (help_one()) continue;
      std::unique_lock<std::mutex> lk(mu_);
      if (stop_) return;
      cv_.wait_for(lk, std::chrono::milliseconds(2), [&] {
        if (stop_) return true;
        for (Job* j : jobs_) if (j->next.load() < j->n) return true;
        return false;
      });
      if (stop_) return;
    }
  }
  std::vector<std::thread> workers_;
  std::mutex mu_;
  std::condition_variable cv_;
  std::vector<Job*> jobs_;
  bool stop_ = false;
};

// Run f(k) for k in [0, n) on the worker pool (callable from inside a task).
template <class F>
void parallel_for(uint32_t n, F f) {
  if (n <= 1) { if (n) f(0); return; }
  std::function<void(uint32_t)> job = [&](uint32_t k) { f(k); };
  Pool::get().run(n, job);
}

// Run f(lo, hi) over [0, n) split into ranges of about `grain` items, in parallel.
template <class F>
void parallel_ranges(uint64_t n, uint64_t grain, F f) {
  const uint64_t parts = (n + grain - 1) / grain;
  if (parts <= 1) { if (n) f(0, n); return; }
  parallel_for((uint32_t)parts, [&](uint32_t i) { f(i * grain, std::min(n, (i + 1) * grain)); });
}

// Deterministic error reporting from parallel validation: the lowest failing index wins.
struct FirstErr {
  std::mutex mu;
  uint64_t idx = UINT64_MAX;
  gdroid_status st = GDROID_OK;
  std::string msg;
  void offer(uint64_t i, gdroid_status s) {
    std::lock_guard<std::mutex> l(mu);
    if (i < idx) { idx = i; st = s; msg = g_err; }
  }
  gdroid_status result() {
    if (st != GDROID_OK) g_err = msg;
    return st;
  }
};

// Call f(i) for every non-zero byte of a (sparse) mark table, in index order.
template <class F>
void scan_marks(const std::vector<uint8_t>& mark, F f) {
  const uint64_t n = mark.size();
  uint64_t i = 0;
  for (; i + 8 <= n; i += 8) {
    uint64_t w;
    std::memcpy(&w, mark.data() + i, 8);
    while (w) {
      const int b = __builtin_ctzll(w) >> 3;
      f(i + b);
      w &= ~(0xffull << (8 * b));
    }
  }
  for (; i < n; ++i)
    if (mark[i]) f(i);
}

// dl = true (device layout, layout.cu): only the per-type / per-method / per-module part and the
// O(1) CSR bounds run here; the per-node and per-edge passes (CSR checks, node pass, projection
// tables, edge pass) are the layout kernels' work.
gdroid_status add_app(HostImage& H, const gdroid_icfg_desc* d, uint32_t k, bool dl = false) {
  if (!d) return set_err(GDROID_E_INVALID, "app %u: NULL descriptor", k);
  if (d->abi_version != GDROID_ABI_VERSION)
    return set_err(GDROID_E_INVALID, "app %u: abi_version %u != %u", k, d->abi_version, GDROID_ABI_VERSION);
  const uint64_t N = d->n_nodes, E = d->n_edges, M = d->n_methods, Dm = d->n_modules;
  const uint64_t I = d->n_instances, G = d->n_statics, T = d->n_types;
  if (N == 0 || M == 0 || Dm == 0 || I == 0) return set_err(GDROID_E_INVALID, "app %u: empty ICFG", k);
  if (N >= (1ull << 32) || E >= (1ull << 32))
    return set_err(GDROID_E_LIMIT, "app %u: batch exceeds 2^32 nodes or edges", k);
  if (!dl) H.args.reserve(H.args.size() + d->call_arg_ptr[N]);
  const uint32_t nb = 0, mb = (uint32_t)H.meths.size();   // app-local node / method indices
  const uint32_t db = (uint32_t)H.mods.size(), tb = (uint32_t)(H.tf_ptr.size() - 1);
  // ---- CSR (structure)
  if (d->row_ptr[0] != 0) return set_err(GDROID_E_INVALID, "app %u: row_ptr[0] != 0", k);
  if (dl && d->row_ptr[N] != E) return set_err(GDROID_E_INVALID, "app %u: row_ptr[n_nodes] != n_edges", k);
  if (!dl) {
    FirstErr fc;                                             // parallel over ranges; lowest index wins
    parallel_ranges(N, 1 << 16, [&](uint64_t lo, uint64_t hi) {
      for (uint64_t n = lo; n < hi; ++n) {
        if (d->row_ptr[n + 1] < d->row_ptr[n]) { fc.offer(n, set_err(GDROID_E_INVALID, "app %u: row_ptr not monotone at node %llu", k, (unsigned long long)n)); return; }
        if (d->node_kind[n] > GK_ASTORE) { fc.offer(n, set_err(GDROID_E_INVALID, "app %u: node %llu bad kind", k, (unsigned long long)n)); return; }
        if (d->node_method[n] >= M) { fc.offer(n, set_err(GDROID_E_INVALID, "app %u: node %llu method out of range", k, (unsigned long long)n)); return; }
      }
    });
    if (fc.st != GDROID_OK) return fc.result();
    if (d->row_ptr[N] != E) return set_err(GDROID_E_INVALID, "app %u: row_ptr[n_nodes] != n_edges", k);
    parallel_ranges(E, 1 << 17, [&](uint64_t lo, uint64_t hi) {
      for (uint64_t e = lo; e < hi; ++e) {
        if (d->col[e] >= N) { fc.offer(N + e, set_err(GDROID_E_INVALID, "app %u: edge %llu target out of range", k, (unsigned long long)e)); return; }
        if (d->edge_kind[e] > GE_C2R) { fc.offer(N + e, set_err(GDROID_E_INVALID, "app %u: edge %llu bad kind", k, (unsigned long long)e)); return; }
      }
    });
    if (fc.st != GDROID_OK) return fc.result();
  }
  PHASE("csr checks");
  // ---- types
  for (uint64_t t = 0; t < T; ++t) {
    if (d->type_field_ptr[t + 1] < d->type_field_ptr[t]) return set_err(GDROID_E_INVALID, "app %u: type_field_ptr not monotone at %llu", k, (unsigned long long)t);
    for (uint64_t q = d->type_field_ptr[t]; q < d->type_field_ptr[t + 1]; ++q) {
      if (d->type_fields[q] >= d->n_fields) return set_err(GDROID_E_INVALID, "app %u: type %llu field out of range", k, (unsigned long long)t);
      if (q > d->type_field_ptr[t] && d->type_fields[q] <= d->type_fields[q - 1])
        return set_err(GDROID_E_INVALID, "app %u: type %llu fields not strictly ascending", k, (unsigned long long)t);
    }
    H.tf_ptr.push_back((uint32_t)(H.tf.size() + (d->type_field_ptr[t + 1] - d->type_field_ptr[t])));
    for (uint64_t q = d->type_field_ptr[t]; q < d->type_field_ptr[t + 1]; ++q) H.tf.push_back(d->type_fields[q]);
  }
  if (d->inst_type[0] != -1) return set_err(GDROID_E_INVALID, "app %u: instance 0 must be NULL (type -1)", k);
  std::vector<uint64_t>& heap_base = H.t_heap_base;
  heap_base.assign(I + 1, 0);
  for (uint64_t o = 0; o < I; ++o) {
    const int32_t t = d->inst_type[o];
    if (t < -1 || t >= (int64_t)T) return set_err(GDROID_E_INVALID, "app %u: instance %llu type out of range", k, (unsigned long long)o);
    heap_base[o + 1] = heap_base[o] + (t < 0 ? 0 : d->type_field_ptr[t + 1] - d->type_field_ptr[t]);
  }
  PHASE("types");
  // ---- methods / slot numbering
  std::vector<uint64_t>& local_base = H.t_local_base;
  local_base.assign(M + 1, 0);
  for (uint64_t m = 0; m < M; ++m) {
    if (d->method_module[m] >= Dm) return set_err(GDROID_E_INVALID, "app %u: method %llu module out of range", k, (unsigned long long)m);
    if (d->method_n_locals[m] < d->method_n_params[m] + 1) return set_err(GDROID_E_INVALID, "app %u: method %llu n_locals < n_params + 1", k, (unsigned long long)m);
    const uint32_t en = d->method_entry[m], ex = d->method_exit[m];
    if (en >= N || d->node_kind[en] != GK_ENTRY || d->node_method[en] != m) return set_err(GDROID_E_INVALID, "app %u: method %llu entry", k, (unsigned long long)m);
    if (ex >= N || d->node_kind[ex] != GK_EXIT || d->node_method[ex] != m) return set_err(GDROID_E_INVALID, "app %u: method %llu exit", k, (unsigned long long)m);
    local_base[m + 1] = local_base[m] + d->method_n_locals[m];
  }
  const uint64_t Lt = local_base[M];
  if (Lt + G + heap_base[I] >= (1ull << 32)) return set_err(GDROID_E_LIMIT, "app %u: more than 2^32 slots", k);
  PHASE("methods");
  // ---- modules: pools, rows, columns (validated and sized in parallel, prefix, filled in parallel)
  std::vector<ModInfo> mi(Dm);
  std::vector<uint64_t>& msz = H.t_msize;                     // per module: cols, heap rows
  msz.assign(2 * Dm + 2, 0);
  {
    FirstErr fm;
    parallel_ranges(Dm, 64, [&](uint64_t lo, uint64_t hi) {
      for (uint64_t dd = lo; dd < hi; ++dd) {
        const uint64_t a = d->module_inst_ptr[dd], b = d->module_inst_ptr[dd + 1];
        const uint64_t sa = d->module_static_ptr[dd], sb = d->module_static_ptr[dd + 1];
        if (b < a || sb < sa) { fm.offer(dd, set_err(GDROID_E_INVALID, "app %u: module %llu pool CSR not monotone", k, (unsigned long long)dd)); return; }
        if (b == a || d->module_insts[a] != 0) { fm.offer(dd, set_err(GDROID_E_POOL, "app %u: module %llu pool lacks NULL", k, (unsigned long long)dd)); return; }
        uint64_t nheap = 0;
        for (uint64_t q = a; q < b; ++q) {
          if (d->module_insts[q] >= I) { fm.offer(dd, set_err(GDROID_E_INVALID, "app %u: module %llu instance out of range", k, (unsigned long long)dd)); return; }
          if (q > a && d->module_insts[q] <= d->module_insts[q - 1]) { fm.offer(dd, set_err(GDROID_E_INVALID, "app %u: module %llu pool not strictly ascending", k, (unsigned long long)dd)); return; }
          const int32_t t = d->inst_type[d->module_insts[q]];
          if (t >= 0) nheap += d->type_field_ptr[t + 1] - d->type_field_ptr[t];
        }
        for (uint64_t q = sa; q < sb; ++q) {
          if (d->module_statics[q] >= G) { fm.offer(dd, set_err(GDROID_E_INVALID, "app %u: module %llu static out of range", k, (unsigned long long)dd)); return; }
          if (q > sa && d->module_statics[q] <= d->module_statics[q - 1]) { fm.offer(dd, set_err(GDROID_E_INVALID, "app %u: module %llu statics not strictly ascending", k, (unsigned long long)dd)); return; }
        }
        if (b - a > 64ull * MAXW) { fm.offer(dd, set_err(GDROID_E_LIMIT, "app %u: module %llu pool has %llu > %d instances", k, (unsigned long long)dd, (unsigned long long)(b - a), 64 * MAXW)); return; }
        msz[2 * dd + 2] = b - a;                                // prefixed below
        msz[2 * dd + 3] = (sb - sa) + nheap;
      }
    });
    if (fm.st != GDROID_OK) return fm.result();
  }
  for (uint64_t dd = 0; dd < Dm; ++dd) {                        // prefix: column / global-row offsets
    msz[2 * dd + 2] += msz[2 * dd];
    msz[2 * dd + 3] += msz[2 * dd + 1];
  }
  const size_t col0 = H.col_gid.size(), grow0 = H.grow_gid.size();
  H.col_gid.resize(col0 + msz[2 * Dm]); H.col_type.resize(col0 + msz[2 * Dm]); H.col_hbase.resize(col0 + msz[2 * Dm]);
  H.grow_gid.resize(grow0 + msz[2 * Dm + 1]); H.grow_col.resize(grow0 + msz[2 * Dm + 1]);
  H.grow_field.resize(grow0 + msz[2 * Dm + 1]);
  H.mods.resize(db + Dm);
  parallel_ranges(Dm, 64, [&](uint64_t lo, uint64_t hi) {
    for (uint64_t dd = lo; dd < hi; ++dd) {
      const uint64_t a = d->module_inst_ptr[dd], b = d->module_inst_ptr[dd + 1];
      const uint64_t sa = d->module_static_ptr[dd], sb = d->module_static_ptr[dd + 1];
      const uint64_t ncol = b - a;
      uint32_t W = 1, logW = 0;
      while (64ull * W < ncol) { W <<= 1; ++logW; }
      ModRec md{};
      md.n_cols = (uint32_t)ncol; md.W = W; md.logW = logW;
      md.n_stat = (uint32_t)(sb - sa);
      md.col_off = (uint32_t)(col0 + msz[2 * dd]);
      md.grow_off = (uint32_t)(grow0 + msz[2 * dd + 1]);
      uint32_t g = md.grow_off;
      for (uint64_t q = sa; q < sb; ++q, ++g) {                // static rows
        H.grow_gid[g] = (uint32_t)(Lt + d->module_statics[q]);
        H.grow_col[g] = -1; H.grow_field[g] = -1;
      }
      uint32_t hrow = md.n_stat;
      for (uint64_t c = 0; c < ncol; ++c) {                    // columns + heap rows
        const uint32_t o = d->module_insts[a + c];
        const int32_t t = d->inst_type[o];
        H.col_gid[md.col_off + c] = o;
        H.col_type[md.col_off + c] = t < 0 ? -1 : (int32_t)(tb + t);
        H.col_hbase[md.col_off + c] = hrow;
        if (t >= 0) {
          for (uint64_t q = d->type_field_ptr[t]; q < d->type_field_ptr[t + 1]; ++q, ++g) {
            H.grow_gid[g] = (uint32_t)(Lt + G + heap_base[o] + (q - d->type_field_ptr[t]));
            H.grow_col[g] = (int32_t)c;
            H.grow_field[g] = (int32_t)d->type_fields[q];
            ++hrow;
          }
        }
      }
      md.n_glob = hrow;
      H.mods[db + dd] = md;
      mi[dd] = ModInfo{d->module_insts + a, ncol, d->module_statics + sa, sb - sa, db + (uint32_t)dd};
    }
  });
  for (uint64_t m = 0; m < M; ++m)
    H.meths.push_back(MethRec{d->method_n_locals[m], d->method_n_params[m], db + d->method_module[m], (uint32_t)local_base[m]});
  PHASE("modules");
  // ---- nodes: operands -> rows (V1, V2, V4), fact offsets (parallel over node ranges)
  H.app_node_base.push_back(nb);
  if (d->call_arg_ptr[0] != 0) return set_err(GDROID_E_INVALID, "app %u: call_arg_ptr[0] != 0", k);
  if (dl) {
    H.n_nodes = N;
    H.n_edges = E;
    H.desc = d;
    for (uint64_t i = 0; i < d->n_entries; ++i) {
      if (d->entries[i] >= N || d->node_kind[d->entries[i]] != GK_ENTRY) return set_err(GDROID_E_INVALID, "app %u: entry %llu is not an ENTRY node", k, (unsigned long long)i);
      H.entries.push_back(nb + d->entries[i]);
    }
    return GDROID_OK;
  }
  // per range: call_arg_ptr monotone, fact-block sizes, (module, field) keys of heap accesses
  constexpr uint64_t RG = 1 << 15;
  const uint64_t n_rg = (N + RG - 1) / RG;
  auto& foff = H.t_foff;
  foff.resize(N + 1);
  foff[0] = 0;
  std::vector<uint64_t> rg_sum(n_rg + 1, 0);
  std::vector<std::vector<uint64_t>> rg_keys(n_rg);
  // (module, field) keys of heap accesses: a dense mark table when Dm x n_fields is small,
  // else per-range sorted key lists merged below
  const uint64_t NF = d->n_fields;
  const bool force_sparse = getenv("GDROID_LOADER_SPARSE") != nullptr;   // tests: sorted-key paths
  const bool kdense = !force_sparse && (uint64_t)Dm * NF <= (1ull << 22);
  std::vector<uint8_t>& kmark = H.t_kmark;
  if (kdense) kmark.assign(Dm * NF, 0);
  FirstErr fe0;
  auto fkey = [&](uint64_t n) -> uint64_t {                 // UINT64_MAX: no field-row table
    const uint8_t kind = d->node_kind[n];
    if (kind != GK_FLOAD && kind != GK_ALOAD && kind != GK_FSTORE && kind != GK_ASTORE) return UINT64_MAX;
    const int32_t f = (kind == GK_ALOAD || kind == GK_ASTORE) ? (int32_t)GDROID_F_ARR : d->node_ops[4 * n + 2];
    if (f < 0 || (uint32_t)f >= d->n_fields) return UINT64_MAX;   // reported by the node pass
    return ((uint64_t)d->method_module[d->node_method[n]] << 32) | (uint32_t)f;
  };
  parallel_ranges(N, RG, [&](uint64_t lo, uint64_t hi) {
    uint64_t acc = 0;
    std::vector<uint64_t>& keys = rg_keys[lo / RG];
    for (uint64_t n = lo; n < hi; ++n) {
      if (d->call_arg_ptr[n + 1] < d->call_arg_ptr[n]) {
        set_err(GDROID_E_INVALID, "app %u: call_arg_ptr not monotone at %llu", k, (unsigned long long)n);
        fe0.offer(n, GDROID_E_INVALID);
        return;
      }
      const uint64_t m = d->node_method[n];
      const ModRec& md = H.mods[db + d->method_module[m]];
      const uint64_t rows = d->method_n_locals[m] + md.n_glob;
      uint64_t w = ((rows << md.logW) + 3) & ~3ull;            // 32-byte aligned blocks
      if (md.logW >= 1) w += (((rows + 63) >> 6) + 3) & ~3ull;  // wide: row-occupancy words
      acc += w;
      foff[n + 1] = acc;                                       // range-local inclusive prefix
      const uint64_t key = fkey(n);
      if (key != UINT64_MAX) {
        if (kdense) __atomic_store_n(&kmark[(key >> 32) * NF + (uint32_t)key], (uint8_t)1, __ATOMIC_RELAXED);
        else keys.push_back(key);
      }
    }
    rg_sum[lo / RG + 1] = acc;
    if (!kdense) {
      std::sort(keys.begin(), keys.end());
      keys.erase(std::unique(keys.begin(), keys.end()), keys.end());
    }
  });
  if (fe0.st != GDROID_OK) return fe0.result();
  const uint64_t n_args = d->call_arg_ptr[N];
  for (uint64_t r = 0; r < n_rg; ++r) rg_sum[r + 1] += rg_sum[r];
  parallel_ranges(N, RG, [&](uint64_t lo, uint64_t hi) {
    const uint64_t base = rg_sum[lo / RG];
    for (uint64_t n = lo; n < hi; ++n) foff[n + 1] += base;
  });
  PHASE("node sizes + field keys");
  // field-row tables of FLOAD/FSTORE/ALOAD/ASTORE: one per (module, field) pair used
  std::vector<uint64_t> fkeys;                                  // sorted (module << 32 | field)
  std::vector<uint32_t>& kidx = H.t_kidx;                       // dense: key -> index in fkeys
  if (kdense) {
    kidx.resize(Dm * NF);
    scan_marks(kmark, [&](uint64_t i) { kidx[i] = (uint32_t)fkeys.size(); fkeys.push_back(((i / NF) << 32) | (i % NF)); });
  } else {
    for (auto& v : rg_keys) fkeys.insert(fkeys.end(), v.begin(), v.end());
    std::sort(fkeys.begin(), fkeys.end());
    fkeys.erase(std::unique(fkeys.begin(), fkeys.end()), fkeys.end());
  }
  std::vector<uint32_t> fkey_off(fkeys.size() + 1);
  const size_t frow0 = H.frow.size();
  fkey_off[0] = (uint32_t)frow0;
  for (size_t i = 0; i < fkeys.size(); ++i) fkey_off[i + 1] = fkey_off[i] + H.mods[db + (fkeys[i] >> 32)].n_cols;
  H.frow.resize(fkey_off[fkeys.size()]);
  parallel_ranges(fkeys.size(), 256, [&](uint64_t lo, uint64_t hi) {
    for (uint64_t i = lo; i < hi; ++i) {
      const uint64_t dd = fkeys[i] >> 32;
      const uint32_t f = (uint32_t)fkeys[i];
      const ModRec& md = H.mods[db + dd];
      for (uint32_t c = 0; c < md.n_cols; ++c) {
        const int32_t ty = H.col_type[md.col_off + c];
        int32_t row = -1;
        if (c != 0 && ty >= 0)
          for (uint32_t q = H.tf_ptr[ty]; q < H.tf_ptr[ty + 1]; ++q)
            if (H.tf[q] == f) row = (int32_t)(H.col_hbase[md.col_off + c] + (q - H.tf_ptr[ty]));
        H.frow[fkey_off[i] + c] = row;
      }
    }
  });
  auto frow_of = [&](uint64_t n) -> int32_t {
    const uint64_t key = fkey(n);
    if (key == UINT64_MAX) return -1;
    if (kdense) return (int32_t)fkey_off[kidx[(key >> 32) * NF + (uint32_t)key]];
    return (int32_t)fkey_off[std::lower_bound(fkeys.begin(), fkeys.end(), key) - fkeys.begin()];
  };
  auto local_idx = [&](int64_t gid, uint64_t m) -> int64_t {
    if (gid < (int64_t)local_base[m] || gid >= (int64_t)local_base[m + 1]) return -1;
    return gid - (int64_t)local_base[m];
  };
  H.n_nodes = N;
  H.args.resize(n_args);
  FirstErr fe;
  std::mutex cls_mu;
  auto node_pass = [&](uint64_t n, uint32_t* cls_cnt) -> gdroid_status {
    const uint8_t kind = d->node_kind[n];
    const uint64_t m = d->node_method[n];
    const uint64_t dd = d->method_module[m];
    const ModInfo& P = mi[dd];
    const ModRec& md = H.mods[db + dd];
    const uint32_t L = d->method_n_locals[m];
    const int32_t* op = d->node_ops + 4 * n;
    NodeRec R{};
    R.kind = kind; R.cls = (uint8_t)cls_of(kind); R.app = (uint16_t)k;
    R.r0 = R.r1 = R.r2 = R.r3 = -1;
    auto need_local = [&](int32_t gid, int32_t& out, const char* what) -> bool {
      int64_t i = local_idx(gid, m);
      if (i < 0) { set_err(GDROID_E_POOL, "app %u: node %llu: %s is not a local of its method (V4)", k, (unsigned long long)n, what); return false; }
      out = (int32_t)i;
      return true;
    };
    auto static_row = [&](int32_t gid, int32_t& out) -> gdroid_status {
      if (gid < (int64_t)Lt || gid >= (int64_t)(Lt + G)) return set_err(GDROID_E_INVALID, "app %u: node %llu: operand is not a static slot", k, (unsigned long long)n);
      int64_t pos = bsearch_idx<uint32_t>(P.stats, P.n_stats, (uint32_t)(gid - Lt));
      if (pos < 0) return set_err(GDROID_E_POOL, "app %u: node %llu: static not visible in its module (V2)", k, (unsigned long long)n);
      out = (int32_t)(L + pos);
      return GDROID_OK;
    };
    gdroid_status st = GDROID_OK;
    switch (kind) {
      case GK_PRIM:
        if (!need_local(op[0], R.r0, "lhs")) return GDROID_E_POOL;
        break;
      case GK_CONST: case GK_NEW: {
        if (!need_local(op[0], R.r0, "lhs")) return GDROID_E_POOL;
        if (op[3] < 0 || (uint64_t)op[3] >= I) return set_err(GDROID_E_INVALID, "app %u: node %llu: instance out of range", k, (unsigned long long)n);
        if (kind == GK_NEW && op[3] == 0) return set_err(GDROID_E_INVALID, "app %u: node %llu: NEW of NULL", k, (unsigned long long)n);
        int64_t c = bsearch_idx<uint32_t>(P.insts, P.n_insts, (uint32_t)op[3]);
        if (c < 0) return set_err(GDROID_E_POOL, "app %u: node %llu: site instance not in its module pool (V1)", k, (unsigned long long)n);
        R.r3 = (int32_t)c;
        break;
      }
      case GK_COPY:
        if (!need_local(op[0], R.r0, "lhs") || !need_local(op[1], R.r1, "rhs")) return GDROID_E_POOL;
        break;
      case GK_FLOAD: case GK_FSTORE: case GK_ALOAD: case GK_ASTORE:
        if (!need_local(op[0], R.r0, "op0") || !need_local(op[1], R.r1, "op1")) return GDROID_E_POOL;
        if (kind == GK_ALOAD || kind == GK_ASTORE) R.r2 = (int32_t)GDROID_F_ARR;
        else {
          if (op[2] < 0 || (uint32_t)op[2] >= d->n_fields) return set_err(GDROID_E_INVALID, "app %u: node %llu: field out of range", k, (unsigned long long)n);
          R.r2 = op[2];
        }
        R.r3 = frow_of(n);                                   // heap row of (o1, f) per column
        break;
      case GK_SLOAD:
        if (!need_local(op[0], R.r0, "lhs")) return GDROID_E_POOL;
        if ((st = static_row(op[1], R.r1)) != GDROID_OK) return st;
        break;
      case GK_SSTORE:
        if (!need_local(op[1], R.r1, "rhs")) return GDROID_E_POOL;
        if ((st = static_row(op[0], R.r0)) != GDROID_OK) return st;
        break;
      case GK_RETV:
        if (!need_local(op[1], R.r1, "rhs")) return GDROID_E_POOL;
        R.r0 = (int32_t)(L - 1);                                  // RET_m
        break;
      case GK_CALL:
        if (op[0] >= 0 && !need_local(op[0], R.r0, "call lhs")) return GDROID_E_POOL;
        break;
      case GK_RETSITE: {
        const int32_t c = op[3];
        if (c < 0 || (uint64_t)c >= N || d->node_kind[c] != GK_CALL) return set_err(GDROID_E_INVALID, "app %u: node %llu: RETSITE without its CALL", k, (unsigned long long)n);
        if (d->node_method[c] != m || d->node_ops[4ull * c] != op[0]) return set_err(GDROID_E_INVALID, "app %u: node %llu: RETSITE/CALL mismatch", k, (unsigned long long)n);
        if (op[0] >= 0 && !need_local(op[0], R.r0, "call lhs")) return GDROID_E_POOL;
        break;
      }
      default:
        break;
    }
    const uint64_t a0 = d->call_arg_ptr[n], a1 = d->call_arg_ptr[n + 1];
    if (kind != GK_CALL && a1 != a0) return set_err(GDROID_E_INVALID, "app %u: node %llu: arguments on a non-CALL node", k, (unsigned long long)n);
    for (uint64_t q = a0; q < a1; ++q) {
      int32_t row = -1;
      if (d->call_args[q] >= 0 && !need_local(d->call_args[q], row, "argument")) return GDROID_E_POOL;
      H.args[q] = row;
      if (kind == GK_CALL && a1 - a0 <= 3) (&R.r1)[q - a0] = row;   // inline argument rows
    }
    if (kind == GK_ENTRY) R.r1 = (int32_t)d->method_n_params[m];
    const uint64_t words = (uint64_t)(L + md.n_glob) << md.logW;
    if (words >= (1ull << 32)) return set_err(GDROID_E_LIMIT, "app %u: node %llu: fact block too large", k, (unsigned long long)n);
    if (L > 0xffff) return set_err(GDROID_E_LIMIT, "app %u: node %llu: method with > 65535 locals", k, (unsigned long long)n);
    if (md.logW >= 1 && L + md.n_glob > 1024) return set_err(GDROID_E_LIMIT, "app %u: node %llu: wide block with > 1024 rows", k, (unsigned long long)n);
    if (d->row_ptr[n + 1] - d->row_ptr[n] > 32768) return set_err(GDROID_E_LIMIT, "app %u: node %llu: out-degree > 32768", k, (unsigned long long)n);
    R.off = H.fact_words + foff[n];
    R.B = (uint32_t)words; R.L = L; R.n_stat = md.n_stat;
    R.e0 = (uint32_t)d->row_ptr[n]; R.e1 = (uint32_t)d->row_ptr[n + 1];
    R.col_off = md.col_off; R.grow_off = md.grow_off; R.n_cols = (uint16_t)md.n_cols;
    R.logW = (uint8_t)md.logW; R.local_base = (uint32_t)local_base[m];
    H.o_nodes[n] = R;
    H.o_nodemeth[n] = mb + (uint32_t)m;
    H.o_rowptr[n + 1] = (uint32_t)d->row_ptr[n + 1];
    H.o_argptr[n + 1] = (uint32_t)a1;
    cls_cnt[R.cls] += n_chunks_of(R.e1 - R.e0, R.cls, R.logW);     // work items per GRP class
    return GDROID_OK;
  };
  PHASE("field-row tables");
  parallel_ranges(N, 1 << 14, [&](uint64_t lo, uint64_t hi) {
    uint32_t cc[NCLS] = {0, 0, 0, 0, 0};
    for (uint64_t n = lo; n < hi; ++n) {
      const gdroid_status st = node_pass(n, cc);
      if (st != GDROID_OK) { fe.offer(n, st); return; }
    }
    std::lock_guard<std::mutex> l(cls_mu);
    for (int c = 0; c < NCLS; ++c) H.cls_count[c] += cc[c];
  });
  if (fe.st != GDROID_OK) return fe.result();
  H.fact_words += foff[N];
  PHASE("nodes");
  // ---- projection tables: one per (source module, target module) pair with a CALL/RET edge
  // (source module, target module) pairs: a dense mark table when Dm^2 is small, else sorted
  // per-range lists merged
  std::vector<uint64_t> pairs;
  const bool pdense = !force_sparse && (uint64_t)Dm * Dm <= (1ull << 22);
  std::vector<uint8_t>& pmark = H.t_pmark;
  std::vector<uint32_t>& pidx = H.t_pidx;
  if (pdense) pmark.assign(Dm * Dm, 0);
  {
    std::mutex pm;
    parallel_ranges(N, 1 << 15, [&](uint64_t lo, uint64_t hi) {
      std::vector<uint64_t> loc;
      for (uint64_t n = lo; n < hi; ++n) {
        const uint8_t kind = d->node_kind[n];
        if (kind != GK_CALL && kind != GK_EXIT) continue;
        const uint32_t sm = d->method_module[d->node_method[n]];
        for (uint64_t e = d->row_ptr[n]; e < d->row_ptr[n + 1]; ++e) {
          const uint8_t ek = d->edge_kind[e];
          if (ek != GE_CALL && ek != GE_RET) continue;
          const uint32_t dm = d->method_module[d->node_method[d->col[e]]];
          if (dm == sm) continue;
          if (pdense) __atomic_store_n(&pmark[(uint64_t)sm * Dm + dm], (uint8_t)1, __ATOMIC_RELAXED);
          else loc.push_back(((uint64_t)sm << 32) | dm);
        }
      }
      if (pdense) return;
      std::sort(loc.begin(), loc.end());
      loc.erase(std::unique(loc.begin(), loc.end()), loc.end());
      std::lock_guard<std::mutex> l(pm);
      pairs.insert(pairs.end(), loc.begin(), loc.end());
    });
    if (pdense) {
      pidx.resize(Dm * Dm);
      scan_marks(pmark, [&](uint64_t i) { pidx[i] = (uint32_t)pairs.size(); pairs.push_back(((i / Dm) << 32) | (i % Dm)); });
    } else {
      std::sort(pairs.begin(), pairs.end());
      pairs.erase(std::unique(pairs.begin(), pairs.end()), pairs.end());
    }
  }
  std::vector<uint32_t> pair_off(pairs.size() + 1, 0);
  for (size_t i = 0; i < pairs.size(); ++i) {
    const ModRec &ms = H.mods[db + (pairs[i] >> 32)], &mt = H.mods[db + (uint32_t)pairs[i]];
    pair_off[i + 1] = pair_off[i] + ms.n_cols + mt.n_glob + ms.n_glob;   // colmap, rowmap, rowinv
  }
  const size_t xbase = H.xmap.size();
  H.xmap.resize(xbase + pair_off[pairs.size()]);              // uninitialised: each pair fills its own
  parallel_ranges(pairs.size(), 64, [&](uint64_t lo, uint64_t hi) {
    std::vector<int32_t> t2s;
    for (uint64_t i = lo; i < hi; ++i) {
      // π keeps a column iff its instance is in Q_dst and a global row iff
      // its slot is in P_src; tables built by merging the sorted pools
      const uint32_t sm = (uint32_t)(pairs[i] >> 32), dm = (uint32_t)pairs[i];
      const ModRec &ms = H.mods[db + sm], &mt = H.mods[db + dm];
      const ModInfo &Ps = mi[sm], &Pt = mi[dm];
      int32_t* cmap = H.xmap.data() + xbase + pair_off[i];   // src column -> dst column
      std::fill(cmap, H.xmap.data() + xbase + pair_off[i + 1], -1);
      int32_t* rmap = cmap + ms.n_cols;                       // dst global row -> src global row
      t2s.assign(Pt.n_insts, -1);
      for (uint64_t a = 0, b2 = 0; a < Ps.n_insts && b2 < Pt.n_insts;) {
        if (Ps.insts[a] == Pt.insts[b2]) { cmap[a] = (int32_t)b2; t2s[b2] = (int32_t)a; ++a; ++b2; }
        else if (Ps.insts[a] < Pt.insts[b2]) ++a;
        else ++b2;
      }
      for (uint64_t a = 0, b2 = 0; a < Ps.n_stats && b2 < Pt.n_stats;) {
        if (Ps.stats[a] == Pt.stats[b2]) { rmap[b2] = (int32_t)a; ++a; ++b2; }
        else if (Ps.stats[a] < Pt.stats[b2]) ++a;
        else ++b2;
      }
      for (uint32_t ct = 1; ct < mt.n_cols; ++ct) {            // heap rows of shared instances
        const int32_t cs = t2s[ct];
        const int32_t ty = H.col_type[mt.col_off + ct];
        if (cs < 0 || ty < 0) continue;
        const uint32_t nf = H.tf_ptr[ty + 1] - H.tf_ptr[ty];
        const uint32_t gt = H.col_hbase[mt.col_off + ct], gs = H.col_hbase[ms.col_off + cs];
        for (uint32_t q = 0; q < nf; ++q) rmap[gt + q] = (int32_t)(gs + q);
      }
      int32_t* rinv = rmap + mt.n_glob;                        // src global row -> dst global row
      for (uint32_t g = 0; g < mt.n_glob; ++g)
        if (rmap[g] >= 0) rinv[rmap[g]] = (int32_t)g;
    }
  });
  PHASE("projection tables");
  // ---- edges (V5, V6), parallel over source-node ranges
  H.desc = d;
  H.n_edges = E;
  H.xo.resize(E);
  auto edge_pass = [&](uint64_t n) -> gdroid_status {
    const uint8_t kind = d->node_kind[n];
    const uint64_t m = d->node_method[n];
    int n_c2r = 0;
    for (uint64_t e = d->row_ptr[n]; e < d->row_ptr[n + 1]; ++e) {
      const uint32_t s = d->col[e];
      const uint8_t ek = d->edge_kind[e];
      uint32_t xoff = NO_XMAP;
      switch (ek) {
        case GE_INTRA:
          if (kind == GK_CALL || kind == GK_EXIT || d->node_method[s] != m) return set_err(GDROID_E_INVALID, "app %u: edge %llu: INTRA edge must stay in one method and not leave a CALL/EXIT (V5)", k, (unsigned long long)e);
          break;
        case GE_C2R:
          if (kind != GK_CALL || d->node_kind[s] != GK_RETSITE || d->node_ops[4ull * s + 3] != (int32_t)n) return set_err(GDROID_E_INVALID, "app %u: edge %llu: C2R must join a CALL to its RETSITE (V5)", k, (unsigned long long)e);
          ++n_c2r;
          break;
        case GE_CALL: {
          if (kind != GK_CALL || d->node_kind[s] != GK_ENTRY || d->method_entry[d->node_method[s]] != s) return set_err(GDROID_E_INVALID, "app %u: edge %llu: CALL edge must go from a CALL to a method entry (V5)", k, (unsigned long long)e);
          const uint32_t callee = d->node_method[s];
          if (d->call_arg_ptr[n + 1] - d->call_arg_ptr[n] != d->method_n_params[callee]) return set_err(GDROID_E_INVALID, "app %u: edge %llu: arity mismatch (V6)", k, (unsigned long long)e);
          break;
        }
        case GE_RET: {
          if (kind != GK_EXIT || d->node_kind[s] != GK_RETSITE) return set_err(GDROID_E_INVALID, "app %u: edge %llu: RET edge must go from an EXIT to a RETSITE (V5)", k, (unsigned long long)e);
          const uint32_t c = (uint32_t)d->node_ops[4ull * s + 3];
          bool ok = false;
          for (uint64_t e2 = d->row_ptr[c]; e2 < d->row_ptr[c + 1] && !ok; ++e2)
            ok = d->edge_kind[e2] == GE_CALL && d->col[e2] == d->method_entry[m];
          if (!ok) return set_err(GDROID_E_INVALID, "app %u: edge %llu: RET to a site that does not call this method (V5)", k, (unsigned long long)e);
          break;
        }
      }
      if (ek == GE_CALL || ek == GE_RET) {
        const uint32_t sm = d->method_module[m], dm = d->method_module[d->node_method[s]];
        if (sm != dm) {
          const uint64_t key = ((uint64_t)sm << 32) | dm;
          const size_t i = pdense ? pidx[(uint64_t)sm * Dm + dm]
                                  : std::lower_bound(pairs.begin(), pairs.end(), key) - pairs.begin();
          xoff = (uint32_t)(xbase + pair_off[i]);
        }
      }
      H.xo[e] = xoff;
    }
    if (kind == GK_CALL && n_c2r != 1) return set_err(GDROID_E_INVALID, "app %u: node %llu: a CALL needs exactly one C2R edge (V5)", k, (unsigned long long)n);
    return GDROID_OK;
  };
  parallel_ranges(N, 1 << 14, [&](uint64_t lo, uint64_t hi) {
    for (uint64_t n = lo; n < hi; ++n) {
      const gdroid_status st = edge_pass(n);
      if (st != GDROID_OK) { fe.offer(n, st); return; }
    }
  });
  if (fe.st != GDROID_OK) return fe.result();
  PHASE("edges");
  for (uint64_t i = 0; i < d->n_entries; ++i) {
    if (d->entries[i] >= N || d->node_kind[d->entries[i]] != GK_ENTRY) return set_err(GDROID_E_INVALID, "app %u: entry %llu is not an ENTRY node", k, (unsigned long long)i);
    H.entries.push_back(nb + d->entries[i]);
  }
  return GDROID_OK;
}


// Parts up to P_UPLOAD are staged on the host and uploaded; the edge records after it are
// built on the device by k_edges from P_ECOL / P_EKIND / P_EXOFF.
enum PartId { P_NODES, P_NODEMETH, P_ROWPTR, P_ARGPTR,               // region A: per node
              P_METHS, P_MODS, P_ECOL, P_EKIND, P_EXOFF, P_ARGS, P_COLGID, P_COLTYPE, P_COLHB, P_GROWGID,
              P_GROWCOL, P_GROWFLD, P_TFPTR, P_TF, P_XMAP, P_APPBASE, P_ENTRIES, P_FROW, P_BASES,
              P_UPLOAD, P_EDGES = P_UPLOAD, P_INL, NPART };
constexpr int P_REGION_B = P_METHS;

// Device-table layout of a batch inside the staging buffer.
struct Layout {
  size_t off[NPART] = {};
  size_t total = 0;              // device bytes of the tables
  size_t upload = 0;             // staged (host-built) prefix of them
  std::vector<uint32_t> app_base;
  uint64_t fact_words = 0, N = 0, NC = 0, n_entries = 0, n_meths = 0;
  uint32_t cls_count[NCLS] = {0, 0, 0, 0, 0};
  uint32_t wide = 0;            // max logW over the modules
  uint64_t n_edges = 0, n_args = 0, n_frow = 0, n_xmap = 0;   // table lengths (gdroid_debug_tables)
};

// Process-wide pinned staging buffer and per-app host images, reused by every load: in this
// environment first-touch page faults (~1 GB/s) dominate host-side table building otherwise.
struct LoadCache {
  std::mutex mu;
  void* stage = nullptr;         // region B (all tables but the per-node ones)
  size_t cap = 0;
  void* stage_a = nullptr;       // region A (per-node tables, written by the node pass)
  size_t cap_a = 0;
  bool pinned = false, pinned_a = false;
  std::vector<HostImage> img;
  uint64_t* dl_tot = nullptr;    // mapped pinned totals of the device layout (written by k_dl_totals)
  uint64_t* dl_tot_dev = nullptr;
  // device layout: per-device scratch for the raw descriptor arrays and the layout kernels'
  // temporaries, grow-only and reused by every load (loads are serialised by mu and each one
  // waits for its layout kernels), so it never churns the stream-ordered pool between the
  // persistent tables and the fact stores
  void* dl_raw[64] = {};
  size_t dl_raw_cap[64] = {};
};
LoadCache g_cache;

void reset_image(HostImage& h) {
  h.n_nodes = 0; h.meths.clear(); h.mods.clear(); h.xo.clear(); h.n_edges = 0; h.desc = nullptr; h.args.clear();
  h.col_gid.clear(); h.col_hbase.clear(); h.col_type.clear(); h.grow_gid.clear(); h.grow_col.clear();
  h.grow_field.clear(); h.tf.clear(); h.xmap.clear(); h.frow.clear(); h.app_node_base.clear();
  h.entries.clear();
  h.tf_ptr.assign(1, 0);
  h.fact_words = 0;
  for (auto& c : h.cls_count) c = 0;
}

size_t align256(size_t x);

// Build every app's image (in parallel, app-local indices) and write the rebased batch tables
// straight into the pinned staging buffer.  Caller holds g_cache.mu.
// Pinned staging buffer of at least `need` bytes.  Without a usable device (CPU-only hosts run
// the validation tests) it falls back to pageable memory; the upload then fails with the CUDA
// error after validation has reported any input error.
gdroid_status ensure_pinned(void*& buf, size_t& cap, bool& pinned, size_t need, const char* what) {
  if (cap >= need) return GDROID_OK;
  if (buf) { if (pinned) cudaFreeHost(buf); else std::free(buf); }
  buf = nullptr;
  cap = 0;
  const size_t want = need + (need >> 2);
  pinned = cudaMallocHost(&buf, want) == cudaSuccess;
  if (!pinned) {
    cudaGetLastError();
    buf = std::malloc(want);
    if (!buf) return set_err(GDROID_E_OOM, "staging %s (%zu B)", what, need);
  }
  cap = want;
  return GDROID_OK;
}

// Region A of the device tables (per-node parts) for a batch of N nodes.
size_t region_a_layout(uint64_t N, Layout& Lo) {
  const size_t bytes[P_REGION_B] = {N * sizeof(NodeRec), N * 4, (N + 1) * 4, (N + 1) * 4};
  size_t t = 0;
  for (int p = 0; p < P_REGION_B; ++p) { Lo.off[p] = t; t += align256(bytes[p]); }
  return t;
}

// upload_a(Lo): called once region A is complete and the full layout is known (before region B
// is written), so its H2D overlaps the rest of the host work.
gdroid_status build_image(const gdroid_icfg_desc* descs, uint32_t n_apps, Layout& Lo,
                          const std::function<gdroid_status(const Layout&)>& upload_a) {
  if (g_cache.img.size() < n_apps) g_cache.img.resize(n_apps);
  std::vector<HostImage>& img = g_cache.img;
  std::vector<gdroid_status> st(n_apps, GDROID_OK);
  std::vector<std::string> err(n_apps);
  std::vector<uint64_t> nbase(n_apps + 1, 0);
  for (uint32_t k = 0; k < n_apps; ++k) nbase[k + 1] = nbase[k] + descs[k].n_nodes;
  if (nbase[n_apps] >= (1ull << 27)) return set_err(GDROID_E_LIMIT, "batch exceeds 2^27 nodes");
  const size_t a_bytes = region_a_layout(nbase[n_apps], Lo);
  gdroid_status sa = ensure_pinned(g_cache.stage_a, g_cache.cap_a, g_cache.pinned_a, a_bytes, "A");
  if (sa != GDROID_OK) return sa;
  char* SA = (char*)g_cache.stage_a;
  NodeRec* a_nodes = (NodeRec*)(SA + Lo.off[P_NODES]);
  uint32_t* a_nodemeth = (uint32_t*)(SA + Lo.off[P_NODEMETH]);
  uint32_t* a_rowptr = (uint32_t*)(SA + Lo.off[P_ROWPTR]);
  uint32_t* a_argptr = (uint32_t*)(SA + Lo.off[P_ARGPTR]);
  a_rowptr[0] = 0; a_argptr[0] = 0;
  PHASE("staging A");
  PhaseTimer* pt_saved = g_pt;
  if (n_apps > 1) g_pt = nullptr;                           // per-app phases only for single apps
  parallel_for(n_apps, [&](uint32_t k) {                   // apps in parallel, and node ranges inside
    reset_image(img[k]);
    img[k].o_nodes = a_nodes + nbase[k]; img[k].o_nodemeth = a_nodemeth + nbase[k];
    img[k].o_rowptr = a_rowptr + nbase[k]; img[k].o_argptr = a_argptr + nbase[k];
    st[k] = add_app(img[k], &descs[k], k);
    if (st[k] != GDROID_OK) err[k] = g_err;
  });
  g_pt = pt_saved;
  for (uint32_t k = 0; k < n_apps; ++k)
    if (st[k] != GDROID_OK) { g_err = err[k]; return st[k]; }
  PHASE("apps (parallel)");
  struct Base { uint64_t node, edge, meth, mod, col, grow, type, tf, xmap, frow, args, fact, ent; };
  std::vector<Base> b(n_apps + 1);
  b[0] = Base{};
  for (uint32_t k = 0; k < n_apps; ++k) {
    const HostImage& h = img[k];
    b[k + 1] = Base{b[k].node + h.n_nodes, b[k].edge + h.n_edges, b[k].meth + h.meths.size(),
                    b[k].mod + h.mods.size(), b[k].col + h.col_gid.size(), b[k].grow + h.grow_gid.size(),
                    b[k].type + (h.tf_ptr.size() - 1), b[k].tf + h.tf.size(), b[k].xmap + h.xmap.size(),
                    b[k].frow + h.frow.size(), b[k].args + h.args.size(), b[k].fact + h.fact_words,
                    b[k].ent + h.entries.size()};
    for (int c = 0; c < NCLS; ++c) Lo.cls_count[c] += h.cls_count[c];
    for (const ModRec& md : h.mods) Lo.wide = std::max<uint32_t>(Lo.wide, md.logW);
  }
  const Base& T = b[n_apps];
  if (T.node >= (1ull << 27)) return set_err(GDROID_E_LIMIT, "batch exceeds 2^27 nodes");
  if (T.edge >= (1ull << 32) || T.xmap >= (1ull << 32) || T.frow >= (1ull << 31))
    return set_err(GDROID_E_LIMIT, "batch tables exceed 32-bit indices");
  uint64_t nc = 0;
  for (int c = 0; c < NCLS; ++c) nc += Lo.cls_count[c];
  if (nc >= (1ull << 31)) return set_err(GDROID_E_LIMIT, "too many work items");
  Lo.N = T.node; Lo.NC = nc; Lo.n_entries = T.ent; Lo.fact_words = T.fact; Lo.n_meths = T.meth;
  Lo.n_edges = T.edge; Lo.n_args = T.args; Lo.n_frow = T.frow; Lo.n_xmap = T.xmap;
  Lo.app_base.resize(n_apps + 1);
  for (uint32_t k = 0; k <= n_apps; ++k) Lo.app_base[k] = (uint32_t)b[k].node;
  const size_t bytes[NPART] = {
      0, 0, 0, 0,                                            // region A (laid out above)
      T.meth * sizeof(MethRec), T.mod * sizeof(ModRec),
      std::max<uint64_t>(T.edge, 1) * 4, std::max<uint64_t>(T.edge, 1), std::max<uint64_t>(T.edge, 1) * 4,
      std::max<uint64_t>(T.args, 1) * 4, T.col * 4, T.col * 4, T.col * 4, T.grow * 4, T.grow * 4, T.grow * 4,
      (T.type + 1) * 4, std::max<uint64_t>(T.tf, 1) * 4, std::max<uint64_t>(T.xmap, 1) * 4, (n_apps + 1) * 4,
      std::max<uint64_t>(T.ent, 1) * 4, std::max<uint64_t>(T.frow, 1) * 4, n_apps * sizeof(AppBase),
      std::max<uint64_t>(T.edge, 1) * sizeof(Edge), T.node * 4 * sizeof(InlEdge)};
  Lo.total = a_bytes;
  for (int p = P_REGION_B; p < NPART; ++p) {
    if (p == P_UPLOAD) Lo.upload = Lo.total;
    Lo.off[p] = Lo.total;
    Lo.total += align256(bytes[p]);
  }
  sa = upload_a(Lo);
  if (sa != GDROID_OK) return sa;
  sa = ensure_pinned(g_cache.stage, g_cache.cap, g_cache.pinned, Lo.upload - a_bytes, "B");
  if (sa != GDROID_OK) return sa;
  char* S = (char*)g_cache.stage - a_bytes;                  // region B starts at device offset a_bytes
  auto P = [&](int p) { return S + Lo.off[p]; };
  MethRec* g_meths = (MethRec*)P(P_METHS);
  ModRec* g_mods = (ModRec*)P(P_MODS);
  uint32_t* g_ecol = (uint32_t*)P(P_ECOL);
  uint8_t* g_ekind = (uint8_t*)P(P_EKIND);
  uint32_t* g_exoff = (uint32_t*)P(P_EXOFF);
  int32_t* g_args = (int32_t*)P(P_ARGS);
  uint32_t* g_colgid = (uint32_t*)P(P_COLGID);
  int32_t* g_coltype = (int32_t*)P(P_COLTYPE);
  uint32_t* g_colhb = (uint32_t*)P(P_COLHB);
  uint32_t* g_growgid = (uint32_t*)P(P_GROWGID);
  int32_t* g_growcol = (int32_t*)P(P_GROWCOL);
  int32_t* g_growfld = (int32_t*)P(P_GROWFLD);
  uint32_t* g_tfptr = (uint32_t*)P(P_TFPTR);
  uint32_t* g_tf = (uint32_t*)P(P_TF);
  int32_t* g_xmap = (int32_t*)P(P_XMAP);
  uint32_t* g_appbase = (uint32_t*)P(P_APPBASE);
  uint32_t* g_entries = (uint32_t*)P(P_ENTRIES);
  int32_t* g_frow = (int32_t*)P(P_FROW);
  AppBase* g_bases = (AppBase*)P(P_BASES);
  for (uint32_t k = 0; k < n_apps; ++k)
    g_bases[k] = AppBase{b[k].fact, (uint32_t)b[k].edge, (uint32_t)b[k].meth, (uint32_t)b[k].mod, (uint32_t)b[k].col,
                         (uint32_t)b[k].grow, (uint32_t)b[k].frow, (uint32_t)b[k].args, 0u};
  g_tfptr[0] = 0;
  g_args[0] = -1; g_tf[0] = 0; g_xmap[0] = -1; g_entries[0] = 0; g_frow[0] = -1;   // non-empty
  for (uint32_t k = 0; k <= n_apps; ++k) g_appbase[k] = (uint32_t)b[k].node;
  // work units: (app, slice of its nodes / edges) so one big app does not serialise the copy
  constexpr size_t SLICE = 1 << 16;
  struct Unit { uint32_t k, kind; size_t lo, hi; };
  std::vector<Unit> units;
  for (uint32_t k = 0; k < n_apps; ++k) {
    const HostImage& h = img[k];
    for (size_t lo = 0; lo < h.n_edges; lo += SLICE) units.push_back({k, 1, lo, std::min<size_t>(h.n_edges, lo + SLICE)});
    units.push_back({k, 2, 0, 0});
  }
  parallel_for((uint32_t)units.size(), [&](uint32_t u) {
    const Unit U = units[u];
    const HostImage& h = img[U.k];
    const Base& B = b[U.k];
    if (U.kind == 1) {
      for (size_t i = U.lo; i < U.hi; ++i) {
        const uint32_t x = h.xo[i];
        g_exoff[B.edge + i] = x == NO_XMAP ? NO_XMAP : x + (uint32_t)B.xmap;
      }
      std::memcpy(g_ecol + B.edge + U.lo, h.desc->col + U.lo, (U.hi - U.lo) * 4);   // app-local ids
      std::memcpy(g_ekind + B.edge + U.lo, h.desc->edge_kind + U.lo, U.hi - U.lo);
      return;
    }
    for (size_t i = 0; i < h.meths.size(); ++i) { MethRec M = h.meths[i]; M.module += (uint32_t)B.mod; g_meths[B.meth + i] = M; }
    for (size_t i = 0; i < h.mods.size(); ++i) {
      ModRec D = h.mods[i]; D.col_off += (uint32_t)B.col; D.grow_off += (uint32_t)B.grow; g_mods[B.mod + i] = D;
    }
    for (size_t i = 0; i < h.col_gid.size(); ++i) {
      g_colgid[B.col + i] = h.col_gid[i];
      g_coltype[B.col + i] = h.col_type[i] < 0 ? -1 : h.col_type[i] + (int32_t)B.type;
      g_colhb[B.col + i] = h.col_hbase[i];
    }
    std::copy(h.grow_gid.begin(), h.grow_gid.end(), g_growgid + B.grow);
    std::copy(h.grow_col.begin(), h.grow_col.end(), g_growcol + B.grow);
    std::copy(h.grow_field.begin(), h.grow_field.end(), g_growfld + B.grow);
    for (size_t i = 1; i < h.tf_ptr.size(); ++i) g_tfptr[B.type + i] = h.tf_ptr[i] + (uint32_t)B.tf;
    std::copy(h.tf.begin(), h.tf.end(), g_tf + B.tf);
    std::copy(h.xmap.begin(), h.xmap.end(), g_xmap + B.xmap);
    std::copy(h.frow.begin(), h.frow.end(), g_frow + B.frow);
    std::copy(h.args.begin(), h.args.end(), g_args + B.args);
    for (size_t i = 0; i < h.entries.size(); ++i) g_entries[B.ent + i] = h.entries[i] + (uint32_t)B.node;
  });
  PHASE("rebase into staging");
  return GDROID_OK;
}

size_t align256(size_t x) { return (x + 255) & ~size_t(255); }

// Pinned, portable host slots for the per-build stats readback, recycled across handles: the
// D2H copy at the end of a build is then truly asynchronous (a pageable destination would make
// cudaMemcpyAsync return only after the build), and gdroid_free needs no cudaFreeHost (which
// would synchronise the device).  Slabs live for the process.
struct StatsSlots {
  std::mutex m;
  std::vector<DevStats*> free_;
  DevStats* get() {
    std::lock_guard<std::mutex> lk(m);
    if (free_.empty()) {
      constexpr int SLAB = 64;
      void* p = nullptr;
      if (cudaHostAlloc(&p, SLAB * sizeof(DevStats), cudaHostAllocPortable) != cudaSuccess) return nullptr;
      for (int i = SLAB - 1; i >= 0; --i) free_.push_back((DevStats*)p + i);
    }
    DevStats* r = free_.back();
    free_.pop_back();
    *r = DevStats{};
    return r;
  }
  void put(DevStats* p) {
    if (!p) return;
    std::lock_guard<std::mutex> lk(m);
    free_.push_back(p);
  }
};
// Raise the release threshold of the device's default memory pool once, so fact stores freed
// with cudaFreeAsync (gdroid_release_facts) stay reserved and the next cudaMallocAsync of a
// batch reuses them without an OS allocation.
void keep_pool_reserved(int device) {
  static std::mutex m;
  static std::vector<char> done;
  std::lock_guard<std::mutex> lk(m);
  if ((int)done.size() <= device) done.resize(device + 1, 0);
  if (done[device]) return;
  cudaMemPool_t pool;
  if (cudaDeviceGetDefaultMemPool(&pool, device) == cudaSuccess) {
    uint64_t thr = ~0ull;
    cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
  }
  done[device] = 1;
}

StatsSlots& stats_slots() {
  static StatsSlots* s = new StatsSlots();   // never destroyed (pinned slabs outlive static teardown)
  return *s;
}

}  // namespace

struct gdroid_app {
  int device = 0;
  cudaStream_t stream = nullptr;
  uint32_t n_apps = 0;
  std::vector<uint32_t> app_base;     // [n_apps+1] global node id ranges
  Dev D{};
  void* d_tables = nullptr;
  void* d_tables2 = nullptr;          // device layout: field-row + projection tables (sized on the device)
  uint64_t tab_len[9] = {};           // elements of each table (gdroid_debug_tables)
  uint64_t* d_facts = nullptr;        // nullptr after gdroid_release_facts (re-allocated by build)
  uint64_t fact_alloc_bytes = 0;
  size_t fact_block_bytes = 0;        // size of the block behind d_facts (fact cache, facts_free)
  void* d_state = nullptr;            // stamp, queue, counts, stats, bar, digests
  uint32_t cls_count[NCLS] = {};      // work items per GRP class (queue segment sizes)
  DevStats* h_stats = nullptr;        // pinned slot (StatsSlots)
  uint64_t* d_scratch = nullptr;
  size_t scratch_bytes = 0;
  cudaEvent_t ev[4] = {nullptr, nullptr, nullptr, nullptr};
  gdroid_build_stats last{};
  uint64_t h2d_ns = 0;
  uint64_t launches = 0;
  bool built = false, pending = false;
  bool digests_ok = false;            // a build completed (digests readable even if facts released)
  uint64_t build_serial = 0;          // completed builds (readback count cache key)
  // incremental builds / out-of-core sub-graphs
  bool state_valid = false;           // stamps hold a completed build's history
  bool mask_stale = false;            // facts imported: narrow occupancy masks must be rebuilt
  bool facts_valid = false;           // the fact store holds facts (build or import), not garbage
  uint32_t round_base = 0;            // rounds used by earlier builds of this handle
  std::vector<uint32_t> seed_nodes;   // staged for the next keep_facts build
  std::vector<uint32_t> seed_pairs;   // (node, slot gid, inst gid) triples
  void* h_seed = nullptr;             // pinned staging of the seeds
  void* d_seed = nullptr;
  size_t seed_cap = 0;
  // SBDA schedule state (allocated at the first SBDA build)
  void* d_sbda = nullptr;
  int sbda_blocks = 0;
  uint64_t counts_build = ~0ull;      // build_serial whose per-node counts are in d_scratch
  bool release_pending = false;
  int max_blocks = 0;
  int max_blocks_lo = 0;              // hybrid (large narrow batches): grid of the 3-CTA/SM instantiation
  int n_sms = 0;
  // PLAIN variant (plain.cu): set-based state, present when loaded with gdroid_load_icfg_plain
  PlainDev P{};
  void* d_plain = nullptr;            // uploaded inputs + sets, locks, stamps, queues, scratch, heap
  int plain_blocks = 0;
  bool last_plain = false;            // the last build ran the PLAIN variant (readback from sets)
};

namespace {

void facts_free(int device, uint64_t* p, size_t bytes, cudaStream_t s);

void free_app(gdroid_app* a) {
  if (!a) return;
  int cur = 0;
  cudaGetDevice(&cur);
  cudaSetDevice(a->device);
  if (a->d_tables) cudaFreeAsync(a->d_tables, a->stream);
  if (a->d_tables2) cudaFreeAsync(a->d_tables2, a->stream);
  if (a->d_facts) facts_free(a->device, a->d_facts, a->fact_block_bytes, a->stream);
  if (a->d_state) cudaFreeAsync(a->d_state, a->stream);
  if (a->d_scratch) facts_free(a->device, a->d_scratch, a->scratch_bytes, a->stream);
  if (a->d_plain) cudaFree(a->d_plain);
  if (a->D.trace) cudaFree(a->D.trace);
  if (a->pending || a->h_seed) cudaStreamSynchronize(a->stream);   // copies target host slots
  if (a->d_seed) cudaFreeAsync(a->d_seed, a->stream);
  if (a->d_sbda) cudaFreeAsync(a->d_sbda, a->stream);
  if (a->h_seed) cudaFreeHost(a->h_seed);
  stats_slots().put(a->h_stats);
  for (auto& e : a->ev)
    if (e) cudaEventDestroy(e);
  cudaSetDevice(cur);
  delete a;
}

struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) { cudaGetDevice(&prev); cudaSetDevice(dev); }
  ~DeviceGuard() { if (prev >= 0) cudaSetDevice(prev); }
};

// Stream-ordered allocation (the device's default pool, release threshold raised) with large
// sizes rounded up to one of 8 size classes per octave (<= 12.5 % slack): the batches of a corpus
// differ by a few percent, and equal sizes let the pool hand a freed block straight to the next
// batch on the same stream instead of mapping new memory — a mapping of a wide app's ~30 GB fact
// store stalled the end-to-end pipeline for ~one build.
size_t size_class(size_t bytes) {
  if (bytes < (256ull << 20)) return bytes;
  int b = 63 - __builtin_clzll(bytes);                        // 2^b <= bytes < 2^(b+1)
  const size_t step = 1ull << (b - 3);
  return (bytes + step - 1) / step * step;
}

cudaError_t pool_alloc(void** p, size_t bytes, cudaStream_t s) {
  return cudaMallocAsync(p, size_class(bytes), s);
}

cudaError_t facts_alloc(int, size_t bytes, cudaStream_t s, uint64_t** p, size_t* got) {
  *got = size_class(bytes);
  return cudaMallocAsync((void**)p, *got, s);
}

void facts_free(int, uint64_t* p, size_t, cudaStream_t s) { cudaFreeAsync(p, s); }

gdroid_status ensure_scratch(gdroid_app* a, size_t bytes) {
  if (a->scratch_bytes >= bytes) return GDROID_OK;
  if (a->d_scratch) facts_free(a->device, a->d_scratch, a->scratch_bytes, a->stream);
  a->d_scratch = nullptr;
  a->scratch_bytes = 0;
  size_t got = 0;
  CU(facts_alloc(a->device, bytes, a->stream, &a->d_scratch, &got));   // large: the block cache
  a->scratch_bytes = got;
  return GDROID_OK;
}

gdroid_status ensure_facts(gdroid_app* a) {
  if (a->d_facts) return GDROID_OK;
  const cudaError_t e = facts_alloc(a->device, a->fact_alloc_bytes, a->stream, &a->d_facts, &a->fact_block_bytes);
  if (e != cudaSuccess) return set_err(GDROID_E_OOM, "fact store (%llu B): %s", (unsigned long long)a->fact_alloc_bytes, cudaGetErrorString(e));
  a->D.facts = a->d_facts;
  a->D.delta = a->D.wide ? a->d_facts + std::max<uint64_t>(a->D.n_words, 4) : nullptr;
  a->facts_valid = false;
  return GDROID_OK;
}

gdroid_status ensure_seed_buf(gdroid_app* a, size_t bytes) {
  if (a->seed_cap >= bytes) return GDROID_OK;
  if (a->h_seed) { CU(cudaStreamSynchronize(a->stream)); cudaFreeHost(a->h_seed); a->h_seed = nullptr; }
  if (a->d_seed) { CU(cudaFreeAsync(a->d_seed, a->stream)); a->d_seed = nullptr; }
  a->seed_cap = 0;
  CU(cudaMallocHost(&a->h_seed, bytes));
  CU(cudaMallocAsync(&a->d_seed, bytes, a->stream));
  a->seed_cap = bytes;
  return GDROID_OK;
}

gdroid_status finish_stats(gdroid_app* a, gdroid_build_stats* out) {
  CU(cudaEventSynchronize(a->ev[3]));
  float ms_build = 0, ms_fix = 0;
  CU(cudaEventElapsedTime(&ms_build, a->ev[0], a->ev[3]));
  CU(cudaEventElapsedTime(&ms_fix, a->ev[1], a->ev[2]));
  gdroid_build_stats s{};
  const DevStats& h = *a->h_stats;
  s.rounds = h.rounds; s.node_visits = h.visits; s.alg_bytes = h.alg_bytes; s.dense_bytes = h.dense_bytes;
  s.atomics = h.atomics;
  for (int i = 0; i < 3; ++i) s.hist[i] = h.hist[i];
  s.build_ns = (uint64_t)(ms_build * 1e6); s.fixpoint_ns = (uint64_t)(ms_fix * 1e6);
  s.h2d_ns = a->h2d_ns;
  s.fact_bytes = a->D.n_words * 8;
  s.kernel_launches = a->launches;
  a->last = s;
  a->pending = false;
  a->built = a->d_facts != nullptr;                   // released facts cannot be read back
  a->digests_ok = true;
  ++a->build_serial;
  if (out) *out = s;
  a->round_base += (uint32_t)h.rounds + 2;            // incremental builds continue the numbering
  if (h.seed_err) return set_err(GDROID_E_POOL, "staged seed pair %llu is outside its node's pools (V1-V4)", (unsigned long long)(h.seed_err - 1));
  if (h.limit_hit) return set_err(GDROID_E_LIMIT, "max_rounds exceeded; facts are an under-approximation");
  return GDROID_OK;
}


// ---------------------------------------------------------------------------- device layout
// (a1) with the per-node / per-edge passes on the device (layout.cu).  The host
// validates and lays out the per-type / per-method / per-module tables of every app (add_app with
// dl = true, apps in parallel), stages them plus the raw descriptor arrays in the pinned buffer
// (parallel memcpy), uploads both, and the layout kernels do the rest.  One host round trip sizes
// the field-row / projection tables.  *applicable = false: the batch's dense (module, field) or
// (module, module) tables would be too large — the caller lays it out on the host instead.  A
// validation error found on the device returns GDROID_E_STATE with *dev_err = the error word; the
// caller re-runs the host validator for the exact status and message.
enum DLPart { Q_METHS, Q_MODS, Q_COLGID, Q_COLTYPE, Q_COLHB, Q_GROWGID, Q_GROWCOL, Q_GROWFLD, Q_TFPTR, Q_TF,
              Q_APPBASE, Q_ENTRIES, Q_UPLOAD,                                  // persistent, uploaded
              Q_NODES = Q_UPLOAD, Q_NODEMETH, Q_ROWPTR, Q_ARGPTR, Q_ARGS, Q_EDGES, Q_INL, Q_NPART };
enum DLRaw { W_KIND, W_METH, W_OPS, W_RP, W_AP, W_COL, W_EKIND, W_CARGS, W_MENTRY, W_APPS, W_UPLOAD,
             W_WORDS = W_UPLOAD, W_FOFF, W_KSZ, W_KOFF, W_PSZ, W_POFF, W_SCAN, W_CLS, W_ERR, W_NPART };
constexpr uint64_t DL_MAX_TABLE = 1ull << 27;   // dense key / pair table entries per batch

gdroid_status load_dl(const gdroid_icfg_desc* descs, uint32_t n_apps, gdroid_app* a, Layout& Lo, bool* applicable,
                      unsigned long long* dev_err) {
  *applicable = true;
  *dev_err = DL_NO_ERR;
  if (g_cache.img.size() < n_apps) g_cache.img.resize(n_apps);
  std::vector<HostImage>& img = g_cache.img;
  std::vector<gdroid_status> st(n_apps, GDROID_OK);
  std::vector<std::string> err(n_apps);
  PhaseTimer* pt_saved = g_pt;
  g_pt = nullptr;
  parallel_for(n_apps, [&](uint32_t k) {
    reset_image(img[k]);
    st[k] = add_app(img[k], &descs[k], k, true);
    if (st[k] != GDROID_OK) err[k] = g_err;
  });
  g_pt = pt_saved;
  for (uint32_t k = 0; k < n_apps; ++k)
    if (st[k] != GDROID_OK) { g_err = err[k]; return st[k]; }
  PHASE("apps (per-module tables)");
  struct Base { uint64_t node, edge, args, meth, mod, col, grow, type, tf, ent, key, pair; };
  std::vector<Base> b(n_apps + 1);
  b[0] = Base{};
  uint32_t wide = 0;
  for (uint32_t k = 0; k < n_apps; ++k) {
    const HostImage& h = img[k];
    const gdroid_icfg_desc& d = descs[k];
    b[k + 1] = Base{b[k].node + d.n_nodes, b[k].edge + d.n_edges, b[k].args + d.call_arg_ptr[d.n_nodes],
                    b[k].meth + h.meths.size(), b[k].mod + h.mods.size(), b[k].col + h.col_gid.size(),
                    b[k].grow + h.grow_gid.size(), b[k].type + (h.tf_ptr.size() - 1), b[k].tf + h.tf.size(),
                    b[k].ent + h.entries.size(), b[k].key + (uint64_t)d.n_modules * d.n_fields,
                    b[k].pair + (uint64_t)d.n_modules * d.n_modules};
    for (const ModRec& md : h.mods) wide = std::max<uint32_t>(wide, md.logW);
  }
  const Base& T = b[n_apps];
  if (T.node >= (1ull << 27)) return set_err(GDROID_E_LIMIT, "batch exceeds 2^27 nodes");
  if (T.edge >= (1ull << 32) || T.args >= (1ull << 32)) return set_err(GDROID_E_LIMIT, "batch tables exceed 32-bit indices");
  if (T.key > DL_MAX_TABLE || T.pair > DL_MAX_TABLE) { *applicable = false; return GDROID_OK; }
  const uint64_t N = T.node, E = T.edge;
  // ---- device layout: persistent tables (A) and temporary inputs + scratch (R)
  const size_t qbytes[Q_NPART] = {
      T.meth * sizeof(MethRec), T.mod * sizeof(ModRec), T.col * 4, T.col * 4, T.col * 4, T.grow * 4, T.grow * 4,
      T.grow * 4, (T.type + 1) * 4, std::max<uint64_t>(T.tf, 1) * 4, (n_apps + 1) * 4, std::max<uint64_t>(T.ent, 1) * 4,
      N * sizeof(NodeRec), N * 4, (N + 1) * 4, (N + 1) * 4, std::max<uint64_t>(T.args, 1) * 4,
      std::max<uint64_t>(E, 1) * sizeof(Edge), N * 4 * sizeof(InlEdge)};
  size_t qoff[Q_NPART + 1];
  qoff[0] = 0;
  for (int p = 0; p < Q_NPART; ++p) qoff[p + 1] = qoff[p] + align256(qbytes[p]);
  const uint64_t scan_n = std::max<uint64_t>(std::max<uint64_t>(N, T.key), T.pair);
  const size_t wbytes[W_NPART] = {
      N, N * 4, N * 16, (N + n_apps) * 8, (N + n_apps) * 8, std::max<uint64_t>(E, 1) * 4, std::max<uint64_t>(E, 1),
      std::max<uint64_t>(T.args, 1) * 4, std::max<uint64_t>(T.meth, 1) * 4, n_apps * sizeof(DLApp),
      N * 4, (N + 1) * 8, std::max<uint64_t>(T.key, 1) * 4, (T.key + 1) * 8, std::max<uint64_t>(T.pair, 1) * 4,
      (T.pair + 1) * 8, scan_tmp_words((uint32_t)scan_n) * 8, 256, 8};
  size_t woff[W_NPART + 1];
  woff[0] = 0;
  for (int p = 0; p < W_NPART; ++p) woff[p + 1] = woff[p] + align256(wbytes[p]);
  const size_t up_a = qoff[Q_UPLOAD], up_r = woff[W_UPLOAD];
  gdroid_status s2 = ensure_pinned(g_cache.stage, g_cache.cap, g_cache.pinned, up_a + up_r, "device-layout inputs");
  if (s2 != GDROID_OK) return s2;
  if (!g_cache.dl_tot) {
    if (cudaHostAlloc(&g_cache.dl_tot, 16 * 8, cudaHostAllocMapped | cudaHostAllocPortable) != cudaSuccess ||
        cudaHostGetDevicePointer((void**)&g_cache.dl_tot_dev, g_cache.dl_tot, 0) != cudaSuccess) {
      cudaGetLastError();
      if (g_cache.dl_tot) cudaFreeHost(g_cache.dl_tot);
      g_cache.dl_tot = nullptr;
      return set_err(GDROID_E_OOM, "mapped pinned device-layout totals");
    }
  }
  char* SA = (char*)g_cache.stage;
  char* SR = SA + up_a;
  MethRec* g_meths = (MethRec*)(SA + qoff[Q_METHS]);
  ModRec* g_mods = (ModRec*)(SA + qoff[Q_MODS]);
  uint32_t* g_colgid = (uint32_t*)(SA + qoff[Q_COLGID]);
  int32_t* g_coltype = (int32_t*)(SA + qoff[Q_COLTYPE]);
  uint32_t* g_colhb = (uint32_t*)(SA + qoff[Q_COLHB]);
  uint32_t* g_growgid = (uint32_t*)(SA + qoff[Q_GROWGID]);
  int32_t* g_growcol = (int32_t*)(SA + qoff[Q_GROWCOL]);
  int32_t* g_growfld = (int32_t*)(SA + qoff[Q_GROWFLD]);
  uint32_t* g_tfptr = (uint32_t*)(SA + qoff[Q_TFPTR]);
  uint32_t* g_tf = (uint32_t*)(SA + qoff[Q_TF]);
  uint32_t* g_appbase = (uint32_t*)(SA + qoff[Q_APPBASE]);
  uint32_t* g_entries = (uint32_t*)(SA + qoff[Q_ENTRIES]);
  DLApp* g_apps = (DLApp*)(SR + woff[W_APPS]);
  g_tfptr[0] = 0; g_tf[0] = 0; g_entries[0] = 0;
  for (uint32_t k = 0; k <= n_apps; ++k) g_appbase[k] = (uint32_t)b[k].node;
  for (uint32_t k = 0; k < n_apps; ++k) {
    const gdroid_icfg_desc& d = descs[k];
    const HostImage& h = img[k];
    const uint64_t Lt = h.meths.empty() ? 0 : (uint64_t)h.meths.back().local_base + h.meths.back().n_locals;
    DLApp A{};
    A.key_base = b[k].key; A.pair_base = b[k].pair; A.n_edges = d.n_edges;
    A.node_base = (uint32_t)b[k].node; A.n_nodes = d.n_nodes; A.edge_base = (uint32_t)b[k].edge;
    A.arg_base = (uint32_t)b[k].args; A.n_args = (uint32_t)d.call_arg_ptr[d.n_nodes];
    A.meth_base = (uint32_t)b[k].meth; A.n_meths = d.n_methods; A.mod_base = (uint32_t)b[k].mod; A.n_mods = d.n_modules;
    A.n_fields = d.n_fields; A.n_inst = d.n_instances;
    A.stat_lo = (uint32_t)Lt; A.stat_hi = (uint32_t)(Lt + d.n_statics);
    A.ptr_base = (uint32_t)(b[k].node + k);
    g_apps[k] = A;
  }
  // work units: each app's per-module tables (rebased to batch indices) and slices of its raw
  // per-node / per-edge arrays (plain copies: the values stay app-local)
  constexpr uint64_t SLICE = 1 << 18;
  struct Unit { uint32_t k, part; uint64_t lo, hi; };
  std::vector<Unit> units;
  for (uint32_t k = 0; k < n_apps; ++k) {
    const gdroid_icfg_desc& d = descs[k];
    units.push_back({k, 99u, 0, 0});
    auto add = [&](uint32_t part, uint64_t n) { for (uint64_t lo = 0; lo < n; lo += SLICE) units.push_back({k, part, lo, std::min(n, lo + SLICE)}); };
    add(W_KIND, d.n_nodes); add(W_METH, d.n_nodes); add(W_OPS, d.n_nodes); add(W_RP, d.n_nodes + 1ull);
    add(W_AP, d.n_nodes + 1ull); add(W_COL, d.n_edges); add(W_EKIND, d.n_edges); add(W_CARGS, d.call_arg_ptr[d.n_nodes]);
    add(W_MENTRY, d.n_methods);
  }
  parallel_for((uint32_t)units.size(), [&](uint32_t u) {
    const Unit U = units[u];
    const HostImage& h = img[U.k];
    const gdroid_icfg_desc& d = descs[U.k];
    const Base& B = b[U.k];
    const uint64_t lo = U.lo, n = U.hi - U.lo;
    switch (U.part) {
      case W_KIND: std::memcpy(SR + woff[W_KIND] + B.node + lo, d.node_kind + lo, n); return;
      case W_METH: std::memcpy(SR + woff[W_METH] + 4 * (B.node + lo), d.node_method + lo, 4 * n); return;
      case W_OPS: std::memcpy(SR + woff[W_OPS] + 16 * (B.node + lo), d.node_ops + 4 * lo, 16 * n); return;
      case W_RP: std::memcpy(SR + woff[W_RP] + 8 * (B.node + U.k + lo), d.row_ptr + lo, 8 * n); return;
      case W_AP: std::memcpy(SR + woff[W_AP] + 8 * (B.node + U.k + lo), d.call_arg_ptr + lo, 8 * n); return;
      case W_COL: std::memcpy(SR + woff[W_COL] + 4 * (B.edge + lo), d.col + lo, 4 * n); return;
      case W_EKIND: std::memcpy(SR + woff[W_EKIND] + B.edge + lo, d.edge_kind + lo, n); return;
      case W_CARGS: std::memcpy(SR + woff[W_CARGS] + 4 * (B.args + lo), d.call_args + lo, 4 * n); return;
      case W_MENTRY: std::memcpy(SR + woff[W_MENTRY] + 4 * (B.meth + lo), d.method_entry + lo, 4 * n); return;
      default: break;
    }
    for (size_t i = 0; i < h.meths.size(); ++i) { MethRec M = h.meths[i]; M.module += (uint32_t)B.mod; g_meths[B.meth + i] = M; }
    for (size_t i = 0; i < h.mods.size(); ++i) {
      ModRec D = h.mods[i]; D.col_off += (uint32_t)B.col; D.grow_off += (uint32_t)B.grow; g_mods[B.mod + i] = D;
    }
    for (size_t i = 0; i < h.col_gid.size(); ++i) {
      g_colgid[B.col + i] = h.col_gid[i];
      g_coltype[B.col + i] = h.col_type[i] < 0 ? -1 : h.col_type[i] + (int32_t)B.type;
      g_colhb[B.col + i] = h.col_hbase[i];
    }
    std::copy(h.grow_gid.begin(), h.grow_gid.end(), g_growgid + B.grow);
    std::copy(h.grow_col.begin(), h.grow_col.end(), g_growcol + B.grow);
    std::copy(h.grow_field.begin(), h.grow_field.end(), g_growfld + B.grow);
    for (size_t i = 1; i < h.tf_ptr.size(); ++i) g_tfptr[B.type + i] = h.tf_ptr[i] + (uint32_t)B.tf;
    std::copy(h.tf.begin(), h.tf.end(), g_tf + B.tf);
    for (size_t i = 0; i < h.entries.size(); ++i) g_entries[B.ent + i] = h.entries[i] + (uint32_t)B.node;
  });
  PHASE("staging");
  // ---- upload, phase 1 (sizes), one round trip
  const auto t0 = std::chrono::steady_clock::now();
  if (a->device < 0 || a->device >= 64) return set_err(GDROID_E_INVALID, "device %d", a->device);
  void*& d_raw = g_cache.dl_raw[a->device];
  size_t& raw_cap = g_cache.dl_raw_cap[a->device];
  if (raw_cap < woff[W_NPART]) {
    if (d_raw) { CU(cudaFree(d_raw)); d_raw = nullptr; raw_cap = 0; }
    const size_t want = woff[W_NPART] + (woff[W_NPART] >> 2);
    CU(cudaMalloc(&d_raw, want));
    raw_cap = want;
  }
  CU(pool_alloc(&a->d_tables, qoff[Q_NPART], a->stream));
  char* DA = (char*)a->d_tables;
  char* DR = (char*)d_raw;
  CU(cudaMemcpyAsync(DA, SA, up_a, cudaMemcpyHostToDevice, a->stream));
  CU(cudaMemcpyAsync(DR, SR, up_r, cudaMemcpyHostToDevice, a->stream));
  CU(cudaMemsetAsync(DR + woff[W_KSZ], 0, wbytes[W_KSZ], a->stream));
  CU(cudaMemsetAsync(DR + woff[W_PSZ], 0, wbytes[W_PSZ], a->stream));
  CU(cudaMemsetAsync(DR + woff[W_CLS], 0, 256, a->stream));
  CU(cudaMemsetAsync(DR + woff[W_ERR], 0xff, 8, a->stream));
  DLDev L{};
  L.kind = (const uint8_t*)(DR + woff[W_KIND]); L.meth = (const uint32_t*)(DR + woff[W_METH]);
  L.ops = (const int32_t*)(DR + woff[W_OPS]); L.rp = (const uint64_t*)(DR + woff[W_RP]);
  L.ap = (const uint64_t*)(DR + woff[W_AP]); L.col = (const uint32_t*)(DR + woff[W_COL]);
  L.ekind = (const uint8_t*)(DR + woff[W_EKIND]); L.cargs = (const int32_t*)(DR + woff[W_CARGS]);
  L.mentry = (const uint32_t*)(DR + woff[W_MENTRY]); L.apps = (const DLApp*)(DR + woff[W_APPS]);
  L.n_apps = n_apps; L.N = (uint32_t)N; L.K = T.key; L.P = T.pair;
  L.words = (uint32_t*)(DR + woff[W_WORDS]); L.foff = (uint64_t*)(DR + woff[W_FOFF]);
  L.ksz = (uint32_t*)(DR + woff[W_KSZ]); L.koff = (uint64_t*)(DR + woff[W_KOFF]);
  L.psz = (uint32_t*)(DR + woff[W_PSZ]); L.poff = (uint64_t*)(DR + woff[W_POFF]);
  L.cls = (uint32_t*)(DR + woff[W_CLS]); L.err = (unsigned long long*)(DR + woff[W_ERR]);
  L.meths = (const MethRec*)(DA + qoff[Q_METHS]); L.mods = (const ModRec*)(DA + qoff[Q_MODS]);
  L.col_gid = (const uint32_t*)(DA + qoff[Q_COLGID]); L.col_type = (const int32_t*)(DA + qoff[Q_COLTYPE]);
  L.col_hbase = (const uint32_t*)(DA + qoff[Q_COLHB]); L.grow_gid = (const uint32_t*)(DA + qoff[Q_GROWGID]);
  L.tf_ptr = (const uint32_t*)(DA + qoff[Q_TFPTR]); L.tf = (const uint32_t*)(DA + qoff[Q_TF]);
  L.nodes = (NodeRec*)(DA + qoff[Q_NODES]); L.nodemeth = (uint32_t*)(DA + qoff[Q_NODEMETH]);
  L.rowptr = (uint32_t*)(DA + qoff[Q_ROWPTR]); L.argptr = (uint32_t*)(DA + qoff[Q_ARGPTR]);
  L.args = (int32_t*)(DA + qoff[Q_ARGS]); L.edges = (Edge*)(DA + qoff[Q_EDGES]); L.inl = (InlEdge*)(DA + qoff[Q_INL]);
  cudaError_t e = launch_dl_sizes(L, (uint64_t*)(DR + woff[W_SCAN]), a->stream);
  if (e != cudaSuccess) return set_err(GDROID_E_CUDA, "layout kernels (sizes): %s", cudaGetErrorString(e));
  // [0] fact words [1] frow [2] xmap [3] err [4..6] class counts: stored into the mapped pinned
  // words by a kernel (posted PCIe writes), not by copies — a copy would queue behind the
  // previous batch's fact readback on the D2H engine
  volatile uint64_t* tot = g_cache.dl_tot;
  e = launch_dl_totals(L, g_cache.dl_tot_dev, a->stream);
  if (e != cudaSuccess) return set_err(GDROID_E_CUDA, "layout totals: %s", cudaGetErrorString(e));
  CU(cudaStreamSynchronize(a->stream));
  a->h2d_ns = (uint64_t)std::chrono::duration_cast<std::chrono::nanoseconds>(std::chrono::steady_clock::now() - t0).count();
  PHASE("upload + layout sizes");
  if (tot[3] != DL_NO_ERR) { *dev_err = tot[3]; return GDROID_E_STATE; }
  const uint64_t fact_words = tot[0], n_frow = tot[1], n_xmap = tot[2];
  uint32_t cls_count[NCLS];
  for (int c = 0; c < NCLS; ++c) cls_count[c] = (uint32_t)(tot[4 + c / 2] >> (32 * (c & 1)));
  uint64_t nc = 0;
  for (int c = 0; c < NCLS; ++c) nc += cls_count[c];
  if (nc >= (1ull << 31)) return set_err(GDROID_E_LIMIT, "too many work items");
  if (n_xmap >= (1ull << 32) || n_frow >= (1ull << 31)) return set_err(GDROID_E_LIMIT, "batch tables exceed 32-bit indices");
  // ---- field-row + projection tables, phase 2
  const size_t fb = align256(std::max<uint64_t>(n_frow, 1) * 4), xb = align256(std::max<uint64_t>(n_xmap, 1) * 4);
  CU(pool_alloc(&a->d_tables2, fb + xb, a->stream));
  L.frow = (int32_t*)a->d_tables2;
  L.xmap = (int32_t*)((char*)a->d_tables2 + fb);
  e = launch_dl_records(L, a->stream);
  if (e != cudaSuccess) return set_err(GDROID_E_CUDA, "layout kernels (records): %s", cudaGetErrorString(e));
  e = launch_dl_totals(L, g_cache.dl_tot_dev, a->stream);
  if (e != cudaSuccess) return set_err(GDROID_E_CUDA, "layout totals: %s", cudaGetErrorString(e));
  CU(cudaStreamSynchronize(a->stream));
  PHASE("layout records");
  if (tot[3] != DL_NO_ERR) { *dev_err = tot[3]; return GDROID_E_STATE; }
  // ---- the handle's view
  Lo.N = N; Lo.NC = nc; Lo.n_entries = T.ent; Lo.fact_words = fact_words; Lo.n_meths = T.meth; Lo.wide = wide;
  Lo.n_edges = E; Lo.n_args = T.args; Lo.n_frow = n_frow; Lo.n_xmap = n_xmap;
  for (int c = 0; c < NCLS; ++c) Lo.cls_count[c] = cls_count[c];
  Lo.app_base.resize(n_apps + 1);
  for (uint32_t k = 0; k <= n_apps; ++k) Lo.app_base[k] = (uint32_t)b[k].node;
  Dev& D = a->D;
  D.nodes = L.nodes; D.meths = L.meths; D.mods = L.mods; D.row_ptr = L.rowptr; D.edges = L.edges;
  D.arg_ptr = L.argptr; D.args = L.args; D.col_gid = L.col_gid; D.col_type = L.col_type; D.col_hbase = L.col_hbase;
  D.grow_gid = L.grow_gid; D.grow_col = (const int32_t*)(DA + qoff[Q_GROWCOL]);
  D.grow_field = (const int32_t*)(DA + qoff[Q_GROWFLD]); D.tf_ptr = L.tf_ptr; D.tf = L.tf; D.xmap = L.xmap;
  D.app_node_base = (const uint32_t*)(DA + qoff[Q_APPBASE]); D.entries = (const uint32_t*)(DA + qoff[Q_ENTRIES]);
  D.node_method = L.nodemeth; D.frow = L.frow; D.inl = L.inl;
  return GDROID_OK;
}

// A validation error found by the layout kernels: the host validator (the host layout path)
// re-runs on the batch for the exact status and message of the first offending index.
// GDROID_DL_DEVICE_ERRORS=1 reports the device's own finding instead (tests of the kernels' checks).
gdroid_status dl_error(const gdroid_icfg_desc* descs, uint32_t n_apps, unsigned long long w) {
  const uint32_t k = (uint32_t)(w >> 44);
  const unsigned long long idx = (w >> 4) & ((1ull << 40) - 1);
  const int code = (int)(w & 15);
  if (!getenv("GDROID_DL_DEVICE_ERRORS")) {
    Layout L2;
    const gdroid_status st = build_image(descs, n_apps, L2, [](const Layout&) { return GDROID_OK; });
    if (st != GDROID_OK) return st;
  }
  return set_err((gdroid_status)(-code), "app %u: index %llu: %s (device layout validation)", k, idx,
                 code == 2 ? "pool closure violated (V1-V4)" : code == 8 ? "size limit" : "invalid structure (CSR, kinds, V5, V6)");
}

// Device layout unless GDROID_HOST_LAYOUT is set or there is no device (CPU-only hosts run the
// host validator, then fail at the upload).
bool use_device_layout() {
  if (getenv("GDROID_HOST_LAYOUT")) return false;
  int n = 0;
  if (cudaGetDeviceCount(&n) != cudaSuccess) { cudaGetLastError(); return false; }
  return n > 0;
}

// ---------------------------------------------------------------------------------- PLAIN
// Upload one app's descriptor arrays for the set-based plain variant (plain.cu) and size its
// state: per-thread scratch of 3 x maxset pairs (maxset bounds every set a thread holds:
// IN(n), f(IN(n)), an edge image, FSTORE's generated pairs) and the bump-allocated heap.
gdroid_status load_plain(gdroid_app* a, const gdroid_icfg_desc* d) {
  const uint64_t N = d->n_nodes, E = d->n_edges, M = d->n_methods, Dm = d->n_modules, I = d->n_instances,
                 T = d->n_types;
  const uint64_t n_args = d->call_arg_ptr[N], n_insts = d->module_inst_ptr[Dm], n_stat = d->module_static_ptr[Dm],
                 n_tf = d->type_field_ptr[T];
  std::vector<uint64_t> local_base(M + 1, 0), heap_base(I + 1, 0);
  for (uint64_t m = 0; m < M; ++m) local_base[m + 1] = local_base[m] + d->method_n_locals[m];
  for (uint64_t o = 0; o < I; ++o) {
    const int32_t t = d->inst_type[o];
    heap_base[o + 1] = heap_base[o] + (t < 0 ? 0 : d->type_field_ptr[t + 1] - d->type_field_ptr[t]);
  }
  // |P_m| x |Q_m| (+ |Q_m|^2 for FSTORE's generated pairs), max over methods
  std::vector<uint64_t> mod_heap(Dm, 0);
  for (uint64_t q = 0; q < Dm; ++q)
    for (uint64_t k = d->module_inst_ptr[q]; k < d->module_inst_ptr[q + 1]; ++k)
      mod_heap[q] += heap_base[d->module_insts[k] + 1] - heap_base[d->module_insts[k]];
  uint64_t maxset = 8, dense_bound = 0;
  for (uint64_t m = 0; m < M; ++m) {
    const uint32_t q = d->method_module[m];
    const uint64_t Q = d->module_inst_ptr[q + 1] - d->module_inst_ptr[q];
    const uint64_t Pm = d->method_n_locals[m] + (d->module_static_ptr[q + 1] - d->module_static_ptr[q]) + mod_heap[q];
    maxset = std::max(maxset, (Pm + Q) * Q);
  }
  for (uint64_t n = 0; n < N; ++n) {
    const uint32_t q = d->method_module[d->node_method[n]];
    const uint64_t Q = d->module_inst_ptr[q + 1] - d->module_inst_ptr[q];
    dense_bound += (d->method_n_locals[d->node_method[n]] + (d->module_static_ptr[q + 1] - d->module_static_ptr[q]) +
                    mod_heap[q]) * Q;
  }
  // layout of one device allocation
  size_t off = 0;
  auto take = [&](size_t bytes) { size_t o = off; off = align256(off + bytes); return o; };
  const size_t o_rp = take((N + 1) * 8), o_col = take(E * 4), o_ek = take(E), o_nk = take(N), o_nm = take(N * 4),
               o_ops = take(N * 16), o_ap = take((N + 1) * 8), o_args = take(n_args * 4), o_lb = take((M + 1) * 8),
               o_np = take(M * 4), o_mm = take(M * 4), o_ip = take((Dm + 1) * 8), o_is = take(n_insts * 4),
               o_sp = take((Dm + 1) * 8), o_ss = take(n_stat * 4), o_it = take(I * 4), o_tp = take((T + 1) * 8),
               o_tf = take(n_tf * 4), o_hb = take((I + 1) * 8), o_en = take((size_t)d->n_entries * 4);
  // CELL variant tables: per-method matrix geometry, node index inside its
  // method, each method's node list and each module's global-row gids in ascending order
  std::vector<uint32_t> m_rows(M), m_cols(M), m_wpc(M), nidx(N), mcount(M, 0), mnode_ptr(M + 1, 0), mnodes(N);
  std::vector<uint64_t> m_coff(M);
  for (uint64_t n = 0; n < N; ++n) nidx[n] = mcount[d->node_method[n]]++;
  for (uint64_t m = 0; m < M; ++m) mnode_ptr[m + 1] = mnode_ptr[m] + mcount[m];
  for (uint64_t n = 0; n < N; ++n) mnodes[mnode_ptr[d->node_method[n]] + nidx[n]] = (uint32_t)n;
  std::vector<uint32_t> mgrow_ptr(Dm + 1, 0), mgrow;
  for (uint64_t q = 0; q < Dm; ++q) {
    for (uint64_t k = d->module_static_ptr[q]; k < d->module_static_ptr[q + 1]; ++k)
      mgrow.push_back((uint32_t)(local_base[M] + d->module_statics[k]));
    for (uint64_t k = d->module_inst_ptr[q]; k < d->module_inst_ptr[q + 1]; ++k) {
      const uint32_t o = d->module_insts[k];
      for (uint64_t f = heap_base[o]; f < heap_base[o + 1]; ++f)
        mgrow.push_back((uint32_t)(local_base[M] + d->n_statics + f));
    }
    mgrow_ptr[q + 1] = (uint32_t)mgrow.size();
  }
  uint64_t cell_words = 0;
  for (uint64_t m = 0; m < M; ++m) {
    const uint32_t q = d->method_module[m];
    m_rows[m] = d->method_n_locals[m] + (mgrow_ptr[q + 1] - mgrow_ptr[q]);
    m_cols[m] = (uint32_t)(d->module_inst_ptr[q + 1] - d->module_inst_ptr[q]);
    m_wpc[m] = std::max<uint32_t>(1, (mcount[m] + 63) / 64);
    m_coff[m] = cell_words;
    cell_words += (uint64_t)m_rows[m] * m_cols[m] * m_wpc[m];
  }
  const size_t o_mrows = take(M * 4), o_mcols = take(M * 4), o_mwpc = take(M * 4), o_mcoff = take(M * 8),
               o_nidx = take(N * 4), o_mnp = take((M + 1) * 4), o_mnodes = take(N * 4),
               o_mgp = take((Dm + 1) * 4), o_mg = take(std::max<size_t>(mgrow.size(), 1) * 4);
  const size_t in_bytes = off;
  const size_t o_cells = take(std::max<uint64_t>(cell_words, 1) * 8);
  const size_t o_sets = take(N * sizeof(SetDesc)), o_locks = take(N * 4), o_stamp = take(N * 4),
               o_queue = take(3 * N * 4), o_counts = take(256), o_bar = take(256), o_err = take(256),
               o_top = take(256);
  size_t free_b = 0, total_b = 0;
  CU(cudaMemGetInfo(&free_b, &total_b));
  int blocks = plain_max_blocks(a->device);
  const size_t per_thread = 3 * maxset * 8;
  const size_t scratch_budget = std::min<size_t>(free_b / 4, (size_t)32 << 30);
  while (blocks > 1 && (size_t)blocks * 128 * per_thread > scratch_budget) blocks /= 2;
  const size_t o_scr = take((size_t)blocks * 128 * per_thread);
  const size_t heap_bytes = std::max<size_t>((size_t)64 << 20,
      std::min<size_t>((free_b > off ? (free_b - off) / 2 : 0), (size_t)dense_bound * 8 * 4 + ((size_t)16 << 20)));
  const size_t o_heap = take(heap_bytes);
  void* mem = nullptr;
  cudaError_t e = cudaMalloc(&mem, off);
  if (e != cudaSuccess) return set_err(GDROID_E_OOM, "plain state (%zu B): %s", off, cudaGetErrorString(e));
  a->d_plain = mem;
  char* B = (char*)mem;
  std::vector<char> h(in_bytes, 0);
  auto put = [&](size_t o, const void* src, size_t bytes) { if (bytes) std::memcpy(h.data() + o, src, bytes); };
  put(o_rp, d->row_ptr, (N + 1) * 8); put(o_col, d->col, E * 4); put(o_ek, d->edge_kind, E);
  put(o_nk, d->node_kind, N); put(o_nm, d->node_method, N * 4); put(o_ops, d->node_ops, N * 16);
  put(o_ap, d->call_arg_ptr, (N + 1) * 8); put(o_args, d->call_args, n_args * 4);
  put(o_lb, local_base.data(), (M + 1) * 8); put(o_np, d->method_n_params, M * 4); put(o_mm, d->method_module, M * 4);
  put(o_ip, d->module_inst_ptr, (Dm + 1) * 8); put(o_is, d->module_insts, n_insts * 4);
  put(o_sp, d->module_static_ptr, (Dm + 1) * 8); put(o_ss, d->module_statics, n_stat * 4);
  put(o_it, d->inst_type, I * 4); put(o_tp, d->type_field_ptr, (T + 1) * 8); put(o_tf, d->type_fields, n_tf * 4);
  put(o_hb, heap_base.data(), (I + 1) * 8); put(o_en, d->entries, (size_t)d->n_entries * 4);
  put(o_mrows, m_rows.data(), M * 4); put(o_mcols, m_cols.data(), M * 4); put(o_mwpc, m_wpc.data(), M * 4);
  put(o_mcoff, m_coff.data(), M * 8); put(o_nidx, nidx.data(), N * 4); put(o_mnp, mnode_ptr.data(), (M + 1) * 4);
  put(o_mnodes, mnodes.data(), N * 4); put(o_mgp, mgrow_ptr.data(), (Dm + 1) * 4);
  put(o_mg, mgrow.data(), mgrow.size() * 4);
  CU(cudaMemcpy(mem, h.data(), in_bytes, cudaMemcpyHostToDevice));
  PlainDev& P = a->P;
  P.row_ptr = (const uint64_t*)(B + o_rp); P.col = (const uint32_t*)(B + o_col); P.ekind = (const uint8_t*)(B + o_ek);
  P.nkind = (const uint8_t*)(B + o_nk); P.nmeth = (const uint32_t*)(B + o_nm); P.ops = (const int32_t*)(B + o_ops);
  P.arg_ptr = (const uint64_t*)(B + o_ap); P.args = (const int32_t*)(B + o_args);
  P.local_base = (const uint64_t*)(B + o_lb); P.n_params = (const uint32_t*)(B + o_np); P.mmod = (const uint32_t*)(B + o_mm);
  P.inst_ptr = (const uint64_t*)(B + o_ip); P.insts = (const uint32_t*)(B + o_is);
  P.stat_ptr = (const uint64_t*)(B + o_sp); P.statics = (const uint32_t*)(B + o_ss);
  P.inst_type = (const int32_t*)(B + o_it); P.tf_ptr = (const uint64_t*)(B + o_tp); P.tfields = (const uint32_t*)(B + o_tf);
  P.heap_base = (const uint64_t*)(B + o_hb); P.entries = (const uint32_t*)(B + o_en);
  P.L_total = local_base[M]; P.G = d->n_statics;
  P.n_nodes = (uint32_t)N; P.n_instances = (uint32_t)I; P.n_entries = d->n_entries;
  P.sets = (SetDesc*)(B + o_sets); P.locks = (uint32_t*)(B + o_locks); P.stamp = (uint32_t*)(B + o_stamp);
  P.queue = (uint32_t*)(B + o_queue); P.counts = (uint32_t*)(B + o_counts); P.bar = (uint32_t*)(B + o_bar);
  P.err = (uint32_t*)(B + o_err); P.heap_top = (unsigned long long*)(B + o_top);
  P.scratch = (uint64_t*)(B + o_scr); P.maxset = maxset;
  P.heap = (uint64_t*)(B + o_heap); P.heap_cap = heap_bytes / 8;
  P.stats = a->D.stats; P.node_digest = a->D.node_digest; P.app_digest = a->D.app_digest;
  P.cell = 0; P.n_methods = (uint32_t)M;
  P.cells = (uint64_t*)(B + o_cells); P.cell_words = cell_words;
  P.m_rows = (const uint32_t*)(B + o_mrows); P.m_cols = (const uint32_t*)(B + o_mcols);
  P.m_wpc = (const uint32_t*)(B + o_mwpc); P.m_coff = (const uint64_t*)(B + o_mcoff);
  P.nidx = (const uint32_t*)(B + o_nidx); P.mnode_ptr = (const uint32_t*)(B + o_mnp);
  P.mnodes = (const uint32_t*)(B + o_mnodes); P.mgrow_ptr = (const uint32_t*)(B + o_mgp);
  P.mgrow = (const uint32_t*)(B + o_mg);
  a->plain_blocks = blocks;
  return GDROID_OK;
}

// One PLAIN build: zero the sets / worklist state, seed, fixed point, digests (same events
// and stats as the MAT path; alg_bytes = live set bytes, dense_bytes = allocated set bytes
// (Fig. 10 footprint), atomics = array (re)allocations).
gdroid_status build_plain(gdroid_app* a, const gdroid_build_opts& o, gdroid_build_stats* stats) {
  if (!a->d_plain) return set_err(GDROID_E_STATE, "PLAIN / CELL variants need a handle loaded with gdroid_load_icfg_plain");
  PlainDev& P = a->P;
  P.max_rounds = o.max_rounds;
  P.cell = o.variant == GDROID_V_CELL ? 1u : 0u;
  if (P.cell) {
    gdroid_status est = ensure_facts(a);             // the MAT store receives the converted facts
    if (est) return est;
  }
  cudaStream_t s = a->stream;
  const uint32_t N = P.n_nodes;
  a->launches = 0;
  CU(cudaEventRecord(a->ev[0], s));
  CU(cudaMemsetAsync(P.sets, 0, (size_t)N * sizeof(SetDesc), s));
  CU(cudaMemsetAsync(P.locks, 0, (size_t)N * 4, s));
  CU(cudaMemsetAsync(P.stamp, 0, (size_t)N * 4, s));
  CU(cudaMemsetAsync(P.counts, 0, 256, s));
  CU(cudaMemsetAsync(P.bar, 0, 256, s));
  CU(cudaMemsetAsync(P.err, 0, 256, s));
  CU(cudaMemsetAsync(P.heap_top, 0, 256, s));
  CU(cudaMemsetAsync(a->D.stats, 0, sizeof(DevStats), s));
  CU(cudaMemsetAsync(a->D.app_digest, 0, 8, s));
  CU(cudaEventRecord(a->ev[1], s));
  if (P.cell) CU(cudaMemsetAsync(P.cells, 0, P.cell_words * 8, s));
  CU(launch_plain(P, (uint32_t)a->plain_blocks, s));
  a->launches += 2;
  CU(cudaEventRecord(a->ev[2], s));
  if (P.cell) {                                       // cells -> node-major, then the MAT digests
    CU(cudaMemsetAsync(a->D.facts, 0, a->D.n_words * 8, s));
    CU(launch_cell_to_mat(P, a->D, s));
    CU(launch_digest(a->D, s));
    CU(cudaMemsetAsync(&a->D.stats->dense_bytes, 0, 8, s));
    a->launches += 2;
  } else {
    CU(launch_plain_digest(P, s));
    a->launches++;
  }
  CU(cudaEventRecord(a->ev[3], s));
  CU(cudaMemcpyAsync(a->h_stats, a->D.stats, sizeof(DevStats), cudaMemcpyDeviceToHost, s));
  uint32_t err = 0;
  CU(cudaMemcpyAsync(&err, P.err, 4, cudaMemcpyDeviceToHost, s));
  CU(cudaStreamSynchronize(s));
  a->pending = true;
  a->digests_ok = false;
  a->last_plain = !P.cell;                            // CELL reads back from the converted MAT store
  gdroid_status st = finish_stats(a, stats);
  a->last.fact_bytes = P.cell ? P.cell_words * 8 : a->h_stats->dense_bytes;
  if (P.cell) { a->facts_valid = true; a->built = true; }
  if (stats) stats->fact_bytes = a->last.fact_bytes;
  if (err) {
    a->built = false;
    return set_err(GDROID_E_OOM, "PLAIN set heap exhausted (%llu words)", (unsigned long long)P.heap_cap);
  }
  return st;
}

}  // namespace

extern "C" {

gdroid_status gdroid_load_icfg_plain(const gdroid_icfg_desc* desc, int device, void* cuda_stream, gdroid_app** out) {
  gdroid_status st = gdroid_load_batch(desc, 1, device, cuda_stream, out);   // validates; MAT variants too
  if (st != GDROID_OK) return st;
  DeviceGuard guard(device);
  CU(cudaStreamSynchronize((cudaStream_t)cuda_stream));
  st = load_plain(*out, desc);
  if (st != GDROID_OK) { free_app(*out); *out = nullptr; }
  return st;
}


uint32_t gdroid_abi_version(void) { return GDROID_ABI_VERSION; }
const char* gdroid_last_error(void) { return g_err.c_str(); }

gdroid_status gdroid_load_batch(const gdroid_icfg_desc* descs, uint32_t n_apps, int device, void* cuda_stream,
                                gdroid_app** out) {
  if (!out) return set_err(GDROID_E_INVALID, "out is NULL");
  *out = nullptr;
  if (!descs || n_apps == 0 || n_apps > 65535) return set_err(GDROID_E_INVALID, "need 1..65535 apps");
  PhaseTimer pt;
  g_pt = &pt;
  struct Reset { ~Reset() { g_pt = nullptr; } } reset_pt;
  DeviceGuard guard(device);
  gdroid_app* a = new gdroid_app;
  a->device = device;
  a->stream = (cudaStream_t)cuda_stream;
  a->n_apps = n_apps;
  auto fail = [&](gdroid_status st) { free_app(a); return st; };
  {
    // keep freed device memory cached in the stream-ordered pool (handles come and go per batch)
    static bool pool_set[64] = {false};
    if (device >= 0 && device < 64 && !pool_set[device]) {
      cudaMemPool_t pool;
      if (cudaDeviceGetDefaultMemPool(&pool, device) == cudaSuccess) {
        uint64_t thr = UINT64_MAX;
        cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
      }
      pool_set[device] = true;
    }
  }
  Layout Lo;
  auto t0 = std::chrono::steady_clock::now();
  bool dl_done = false;
  if (use_device_layout()) {
    std::lock_guard<std::mutex> lock(g_cache.mu);
    bool applicable = true;
    unsigned long long derr = DL_NO_ERR;
    const gdroid_status st = load_dl(descs, n_apps, a, Lo, &applicable, &derr);
    if (st == GDROID_E_STATE && derr != DL_NO_ERR) return fail(dl_error(descs, n_apps, derr));
    if (st != GDROID_OK) return fail(st);
    dl_done = applicable;
  }
  if (!dl_done) {
    std::lock_guard<std::mutex> lock(g_cache.mu);
    gdroid_status st = build_image(descs, n_apps, Lo, [&](const Layout& L) -> gdroid_status {
      cudaError_t e = pool_alloc(&a->d_tables, L.total, a->stream);
      if (e != cudaSuccess) return set_err(e == cudaErrorMemoryAllocation ? GDROID_E_OOM : GDROID_E_CUDA, "device tables (%zu B): %s", L.total, cudaGetErrorString(e));
      e = cudaMemcpyAsync(a->d_tables, g_cache.stage_a, L.off[P_REGION_B], cudaMemcpyHostToDevice, a->stream);
      return e == cudaSuccess ? GDROID_OK : set_err(GDROID_E_CUDA, "H2D upload (A): %s", cudaGetErrorString(e));
    });
    if (st != GDROID_OK) {
      if (a->d_tables) cudaStreamSynchronize(a->stream);
      return fail(st);
    }
    t0 = std::chrono::steady_clock::now();
    cudaError_t e = cudaMemcpyAsync((char*)a->d_tables + Lo.off[P_REGION_B], g_cache.stage, Lo.upload - Lo.off[P_REGION_B],
                                    cudaMemcpyHostToDevice, a->stream);
    cudaError_t e2 = cudaStreamSynchronize(a->stream);
    if (e != cudaSuccess || e2 != cudaSuccess) return fail(set_err(GDROID_E_CUDA, "H2D upload: %s", cudaGetErrorString(e != cudaSuccess ? e : e2)));
  }
  if (!dl_done) {
    a->h2d_ns = (uint64_t)std::chrono::duration_cast<std::chrono::nanoseconds>(std::chrono::steady_clock::now() - t0).count();
    PHASE("upload");
  }
  a->app_base = Lo.app_base;
  a->tab_len[0] = Lo.N; a->tab_len[1] = Lo.n_edges; a->tab_len[2] = 4 * Lo.N; a->tab_len[3] = Lo.n_frow;
  a->tab_len[4] = Lo.n_xmap; a->tab_len[5] = Lo.n_args; a->tab_len[6] = Lo.N + 1; a->tab_len[7] = Lo.N + 1;
  a->tab_len[8] = Lo.N;
  const uint32_t N = (uint32_t)Lo.N, NC = (uint32_t)Lo.NC;
  char* T = (char*)a->d_tables;
  Dev& D = a->D;
  if (!dl_done) {
  D.nodes = (const NodeRec*)(T + Lo.off[P_NODES]);
  D.meths = (const MethRec*)(T + Lo.off[P_METHS]);
  D.mods = (const ModRec*)(T + Lo.off[P_MODS]);
  D.row_ptr = (const uint32_t*)(T + Lo.off[P_ROWPTR]);
  D.edges = (const Edge*)(T + Lo.off[P_EDGES]);
  D.arg_ptr = (const uint32_t*)(T + Lo.off[P_ARGPTR]);
  D.args = (const int32_t*)(T + Lo.off[P_ARGS]);
  D.col_gid = (const uint32_t*)(T + Lo.off[P_COLGID]);
  D.col_type = (const int32_t*)(T + Lo.off[P_COLTYPE]);
  D.col_hbase = (const uint32_t*)(T + Lo.off[P_COLHB]);
  D.grow_gid = (const uint32_t*)(T + Lo.off[P_GROWGID]);
  D.grow_col = (const int32_t*)(T + Lo.off[P_GROWCOL]);
  D.grow_field = (const int32_t*)(T + Lo.off[P_GROWFLD]);
  D.tf_ptr = (const uint32_t*)(T + Lo.off[P_TFPTR]);
  D.tf = (const uint32_t*)(T + Lo.off[P_TF]);
  D.xmap = (const int32_t*)(T + Lo.off[P_XMAP]);
  D.app_node_base = (const uint32_t*)(T + Lo.off[P_APPBASE]);
  D.entries = (const uint32_t*)(T + Lo.off[P_ENTRIES]);
  D.node_method = (const uint32_t*)(T + Lo.off[P_NODEMETH]);
  D.frow = (const int32_t*)(T + Lo.off[P_FROW]);
  D.inl = (const InlEdge*)(T + Lo.off[P_INL]);
  }
  D.n_nodes = N;
  D.n_chunks = NC;
  D.n_entries = (uint32_t)Lo.n_entries;
  uint32_t acc = 0;
  for (int c = 0; c < NCLS; ++c) { D.seg[c] = acc; acc += Lo.cls_count[c]; a->cls_count[c] = Lo.cls_count[c]; }
  D.seg[NCLS] = acc;
  D.n_words = Lo.fact_words;
  D.wide = Lo.wide;
  D.n_meths = (uint32_t)Lo.n_meths;
  if (!dl_done) {
    // (a1) per-app bases added to the staged app-local node tables, then the edge records and
    // inline chunk-0 edges derived from col / edge_kind / projection offsets and the NodeRecs
    // (stream-ordered after the upload)
    cudaError_t e = launch_rebase(D, (NodeRec*)(T + Lo.off[P_NODES]), (uint32_t*)(T + Lo.off[P_NODEMETH]),
                                  (uint32_t*)(T + Lo.off[P_ROWPTR]), (uint32_t*)(T + Lo.off[P_ARGPTR]),
                                  (const AppBase*)(T + Lo.off[P_BASES]), a->stream);
    if (e != cudaSuccess) return fail(set_err(GDROID_E_CUDA, "k_rebase: %s", cudaGetErrorString(e)));
    e = launch_edges(D, (Edge*)(T + Lo.off[P_EDGES]), (InlEdge*)(T + Lo.off[P_INL]),
                                 (NodeRec*)(T + Lo.off[P_NODES]), (const uint32_t*)(T + Lo.off[P_ECOL]),
                                 (const uint8_t*)(T + Lo.off[P_EKIND]), (const uint32_t*)(T + Lo.off[P_EXOFF]),
                                 a->stream);
    if (e != cudaSuccess) return fail(set_err(GDROID_E_CUDA, "k_edges: %s", cudaGetErrorString(e)));
  }

  // ---- fact store + mutable state
  {
    keep_pool_reserved(device);
    // wide batches: the Δ store of the semi-naive wide path follows the facts (same layout)
    a->fact_alloc_bytes = std::max<uint64_t>(Lo.fact_words, 4) * 8 * (Lo.wide ? 2 : 1);
    cudaError_t e = facts_alloc(device, a->fact_alloc_bytes, a->stream, &a->d_facts, &a->fact_block_bytes);
    if (e != cudaSuccess) return fail(set_err(GDROID_E_OOM, "fact store (%llu B): %s", (unsigned long long)a->fact_alloc_bytes, cudaGetErrorString(e)));
    D.facts = a->d_facts;
    D.delta = Lo.wide ? a->d_facts + std::max<uint64_t>(Lo.fact_words, 4) : nullptr;
    size_t s_mask = GD_NMASK ? align256((size_t)N * 8 * NMW) : 256;
    size_t s_stamp = align256((size_t)N * 8), s_queue = align256((size_t)3 * NC * 4), s_counts = align256(3 * CNT_STRIDE * 4);
    size_t s_stats = align256(sizeof(DevStats)), s_bar = 256, s_nd = align256((size_t)N * 8), s_ad = align256((size_t)n_apps * 8);
    size_t s_pc = align256((size_t)N * 4);
    size_t st = s_mask + s_stamp + s_queue + s_counts + s_stats + s_bar + s_nd + s_ad + s_pc;
    e = pool_alloc(&a->d_state, st, a->stream);
    if (e != cudaSuccess) return fail(set_err(GDROID_E_OOM, "device state (%zu B): %s", st, cudaGetErrorString(e)));
    char* S = (char*)a->d_state;
    D.smask = (uint64_t*)S; S += s_mask;
    D.stamp = (uint32_t*)S;
    D.cont = D.stamp + N; S += s_stamp;
    D.queue = (uint32_t*)S; S += s_queue;
    D.counts = (uint32_t*)S; S += s_counts;
    D.stats = (DevStats*)S; S += s_stats;
    D.bar = (uint32_t*)S; S += s_bar;
    D.node_digest = (uint64_t*)S; S += s_nd;
    D.node_popc = (uint32_t*)S; S += s_pc;
    D.app_digest = (unsigned long long*)S;
    a->h_stats = stats_slots().get();
    if (!a->h_stats) return fail(set_err(GDROID_E_OOM, "pinned stats slot"));
    for (auto& ev : a->ev)
      if (cudaEventCreate(&ev) != cudaSuccess) return fail(set_err(GDROID_E_CUDA, "cudaEventCreate failed"));
  }
  D.hiocc = (D.wide == 0 && N >= HIOCC_NODES) ? 1u : 0u;
  a->max_blocks = fixpoint_max_blocks(device, D.wide, D.hiocc);
  a->max_blocks_lo = fixpoint_max_blocks(device, D.wide, 0u);
  cudaDeviceGetAttribute(&a->n_sms, cudaDevAttrMultiProcessorCount, device);
  PHASE("device state + k_rebase/k_edges");
  *out = a;
  return GDROID_OK;
}

gdroid_status gdroid_load_icfg(const gdroid_icfg_desc* desc, int device, void* cuda_stream, gdroid_app** out) {
  return gdroid_load_batch(desc, 1, device, cuda_stream, out);
}

gdroid_status gdroid_build_idfg(gdroid_app* a, const gdroid_build_opts* opts, gdroid_build_stats* stats) {
  if (!a) return set_err(GDROID_E_INVALID, "app is NULL");
  if (a->pending) return set_err(GDROID_E_STATE, "an async build is still pending; call gdroid_sync");
  gdroid_build_opts o{};
  if (opts) o = *opts;
  DeviceGuard guard(a->device);
  Dev& D = a->D;
  D.max_rounds = o.max_rounds;
  if (o.variant == GDROID_V_PLAIN || o.variant == GDROID_V_CELL) return build_plain(a, o, stats);
  if (o.variant > GDROID_V_SBDA || o.variant == GDROID_V_CELL)
    return set_err(GDROID_E_INVALID, "unknown variant %u", o.variant);
  a->last_plain = false;
  const bool sbda = o.variant == GDROID_V_SBDA;
  static const uint32_t vflags[4] = {F_GRP | F_CONT, 0u, F_GRP, F_GRP | F_MER};
  D.flags = sbda ? F_GRP : vflags[o.variant];
  if (sbda && !a->d_sbda) {                          // method -> nodes CSR, claims, local stamps
    const size_t M = D.n_meths, N = D.n_nodes;
    const size_t bytes = align256((M + 1) * 4) + align256(N * 4) + align256(M * 4) * 2 + align256(N * 8);
    CU(cudaMallocAsync(&a->d_sbda, bytes, a->stream));
    char* S = (char*)a->d_sbda;
    uint32_t* ptr = (uint32_t*)S; S += align256((M + 1) * 4);
    uint32_t* nodes = (uint32_t*)S; S += align256(N * 4);
    uint32_t* cursor = (uint32_t*)S; S += align256(M * 4);
    D.claim = (uint32_t*)S; S += align256(M * 4);
    D.lstamp = (unsigned long long*)S;
    D.meth_node_ptr = ptr;
    D.meth_nodes = nodes;
    CU(launch_meth_csr(D, ptr, nodes, cursor, a->stream));
    a->sbda_blocks = sbda_max_blocks(a->device, D.wide);
  }
  D.count = o.no_byte_model ? 0u : 1u;
  {                                                   // GRP off: one segment holds every item
    uint32_t acc = 0;
    for (int c = 0; c <= NCLS; ++c) {
      D.seg[c] = (D.flags & F_GRP) ? acc : (c == 0 ? 0u : D.n_chunks);
      if (c < NCLS) acc += a->cls_count[c];
    }
  }
  cudaStream_t s = a->stream;
  const uint32_t N = D.n_nodes;
  uint32_t blocks = o.blocks ? std::min<uint32_t>(o.blocks, (uint32_t)a->max_blocks) : (uint32_t)a->max_blocks;
  // reserve_sms: shrink the persistent grids by that share of the SMs (occupancy is per SM)
  auto reserve = [&](uint32_t b) -> uint32_t {
    if (!o.reserve_sms || a->n_sms <= (int)o.reserve_sms) return b;
    const uint64_t r = (uint64_t)b * (uint64_t)(a->n_sms - (int)o.reserve_sms) / (uint64_t)a->n_sms;
    return r ? (uint32_t)r : 1u;
  };
  blocks = reserve(blocks);
  a->launches = 0;
  gdroid_status est = ensure_facts(a);               // released by an earlier build: re-allocate
  if (est) return est;
  // keep_facts (incremental): the fact store keeps its content, the worklist
  // state persists and round numbers continue, so stamps stay ordered and first-reach history
  // is kept; only the staged seeds (plus the entries on a handle's first build) are queued.
  const bool keep = o.keep_facts != 0 && a->state_valid;
  CU(cudaEventRecord(a->ev[0], s));
  // (a2) zero the fact matrices and the worklist state
  if (!(o.keep_facts && a->facts_valid)) CU(cudaMemsetAsync(D.facts, 0, D.n_words * 8, s));
  if (D.delta) CU(cudaMemsetAsync(D.delta, 0, D.n_words * 8, s));   // empty at every fixed point
  const bool facts_kept = o.keep_facts && a->facts_valid;
  if (!keep) {
    CU(cudaMemsetAsync(D.stamp, 0, (size_t)N * 8, s));   // stamp + cont
    if (GD_NMASK) CU(cudaMemsetAsync(D.smask, 0, (size_t)N * 8 * NMW, s));
    a->round_base = 0;
  }
  // narrow word masks must describe the kept facts: rebuilt from them after an import (a fresh
  // handle's masks were just zeroed, the facts were not)
  if (GD_NMASK && facts_kept && (a->mask_stale || !keep)) CU(launch_nmask_rebuild(D, s));
  a->mask_stale = false;
  CU(cudaMemsetAsync(D.counts, 0, 3 * CNT_STRIDE * 4, s));
  CU(cudaMemsetAsync(D.stats, 0, sizeof(DevStats), s));
  CU(cudaMemsetAsync(D.bar, 0, 256, s));                 // barrier + round descriptor words
  CU(cudaMemsetAsync(D.app_digest, 0, (size_t)a->n_apps * 8, s));
  D.round0 = a->round_base + 1;
  D.max_rounds = o.max_rounds ? a->round_base + o.max_rounds : 0u;
  D.push_entries = keep ? 0u : 1u;
  if (o.keep_facts && !a->seed_nodes.empty()) {      // staged seeds -> device (stream-ordered copy)
    const size_t nb = a->seed_nodes.size() * 4, pb = a->seed_pairs.size() * 4;
    gdroid_status st2 = ensure_seed_buf(a, nb + pb + 8);
    if (st2) return st2;
    std::memcpy(a->h_seed, a->seed_nodes.data(), nb);
    std::memcpy((char*)a->h_seed + nb, a->seed_pairs.data(), pb);
    CU(cudaMemcpyAsync(a->d_seed, a->h_seed, nb + pb, cudaMemcpyHostToDevice, s));
    D.seed_nodes = (const uint32_t*)a->d_seed;
    D.seed_pairs = (const uint32_t*)((char*)a->d_seed + nb);
    D.n_seed_nodes = (uint32_t)a->seed_nodes.size();
    D.n_seed_pairs = (uint32_t)(a->seed_pairs.size() / 3);
  } else {
    D.n_seed_nodes = D.n_seed_pairs = 0;
  }
  a->seed_nodes.clear();
  a->seed_pairs.clear();
  CU(launch_seed(D, s));
  a->launches += D.n_seed_pairs ? 2 : 1;
  D.n_seed_nodes = D.n_seed_pairs = 0;
  CU(cudaEventRecord(a->ev[1], s));
  D.sw_lo = D.sw_hi = 0;
  if (!sbda && o.loop_mode == 0 && D.hiocc && GD_HYBRID && (D.flags & F_CONT)) {
    // Hybrid (large narrow batches, default variant): light rounds run in the 3-CTA/SM
    // instantiation with narrow continuation, heavy rounds (>= 4 waves of items) in the 4-CTA/SM
    // one; a launch leaves at the first round of the other kind (bar[3] = that round) and the
    // next launch resumes there.  At most HYB_SWITCHES hand-overs per build.
    // The hand-over is device-side: every launch of the alternating sequence is enqueued up
    // front (no host round trip); a launch starts at the round in bar[3] (k_seed sets 1) and
    // returns at once when bar[3] = 0 (an earlier launch reached the fixed point or the limit).
    uint32_t blocks_lo = reserve(o.blocks ? std::min<uint32_t>(o.blocks, (uint32_t)a->max_blocks_lo) : (uint32_t)a->max_blocks_lo);
    const uint32_t nw_lo = blocks_lo * (THREADS / 32);
    bool heavy = false;
    D.hyb = 1u;
    for (uint32_t sw = 0; sw <= HYB_SWITCHES; ++sw) {
      const bool last = sw == HYB_SWITCHES;
      D.sw_lo = (heavy && !last) ? GD_HYB_LO * nw_lo / 4u : 0u;
      D.sw_hi = (!heavy && !last) ? GD_HYB_HI * nw_lo / 4u : 0u;
      D.hiocc = heavy ? 1u : 0u;
      const cudaError_t e = launch_fixpoint(D, heavy ? blocks : blocks_lo, s);
      D.hiocc = 1u;
      if (e != cudaSuccess) { D.hyb = 0u; return set_err(GDROID_E_CUDA, "k_fixpoint: %s", cudaGetErrorString(e)); }
      a->launches++;
      heavy = !heavy;
    }
    D.hyb = 0u;
    D.sw_lo = D.sw_hi = 0;
  } else if (sbda) {
    CU(cudaMemsetAsync(D.claim, 0, (size_t)D.n_meths * 4, s));
    CU(cudaMemsetAsync(D.lstamp, 0, (size_t)N * 8, s));
    const uint32_t bs = reserve(o.blocks ? std::min<uint32_t>(o.blocks, (uint32_t)a->sbda_blocks) : (uint32_t)a->sbda_blocks);
    CU(launch_sbda(D, bs, s));
    a->launches++;
  } else if (o.loop_mode == 0) {
    CU(launch_fixpoint(D, blocks, s));
    a->launches++;
  } else {
    // one launch per round; the host looks ahead K rounds between termination checks
    const uint32_t K = 64;
    uint32_t* h_counts = nullptr;
    CU(cudaMallocHost(&h_counts, 3 * CNT_STRIDE * 4 + 16));
    uint32_t round = D.round0;
    for (;;) {
      for (uint32_t q = 0; q < K; ++q) {
        cudaError_t e = launch_round(D, round + q, blocks, s);
        if (e != cudaSuccess) { cudaFreeHost(h_counts); return set_err(GDROID_E_CUDA, "k_round: %s", cudaGetErrorString(e)); }
        a->launches++;
      }
      round += K;
      cudaMemcpyAsync(h_counts, D.bar + BAR_DONE, 4, cudaMemcpyDeviceToHost, s);
      cudaError_t e = cudaStreamSynchronize(s);
      if (e != cudaSuccess) { cudaFreeHost(h_counts); return set_err(GDROID_E_CUDA, "round loop: %s", cudaGetErrorString(e)); }
      if (h_counts[0]) break;                                      // a round found an empty worklist
      if (D.max_rounds && round > D.max_rounds + 1) break;
    }
    cudaFreeHost(h_counts);
  }
  CU(cudaEventRecord(a->ev[2], s));
  CU(launch_digest(D, s));
  a->launches++;
  CU(cudaEventRecord(a->ev[3], s));
  CU(cudaMemcpyAsync(a->h_stats, D.stats, sizeof(DevStats), cudaMemcpyDeviceToHost, s));
  a->pending = true;
  a->built = false;
  a->digests_ok = false;
  a->release_pending = o.release_facts != 0;
  a->state_valid = true;
  a->facts_valid = true;
  if (o.release_facts) {                              // stream-ordered: after the digest kernel
    facts_free(a->device, a->d_facts, a->fact_block_bytes, s);
    a->d_facts = nullptr;
    D.facts = D.delta = nullptr;
    a->facts_valid = false;
  }
  if (o.async) return GDROID_OK;
  CU(cudaStreamSynchronize(s));
  return finish_stats(a, stats);
}

gdroid_status gdroid_sync(gdroid_app* a, gdroid_build_stats* stats) {
  if (!a) return set_err(GDROID_E_INVALID, "app is NULL");
  if (!a->pending) return set_err(GDROID_E_STATE, "no pending async build");
  DeviceGuard guard(a->device);
  CU(cudaStreamSynchronize(a->stream));
  return finish_stats(a, stats);
}

// All facts of every app of the batch in one CSR over the batch's nodes (app k's nodes are
// rows app_base[k] .. app_base[k+1]-1, each app's pairs in its own gids).  The size query
// (pairs == NULL) keeps the per-node counts on the device, so the fetch that follows does not
// count again; both copies go straight between the caller's (ideally pinned) buffers and HBM.
gdroid_status gdroid_read_batch_facts(const gdroid_app* ca, uint64_t* ptr, uint64_t* pairs, uint64_t cap) {
  gdroid_app* a = const_cast<gdroid_app*>(ca);
  if (!a) return set_err(GDROID_E_INVALID, "app is NULL");
  if (!a->built) return set_err(GDROID_E_STATE, "facts read before a completed build");
  if (!ptr) return set_err(GDROID_E_INVALID, "ptr is NULL");
  DeviceGuard guard(a->device);
  const uint32_t n = a->app_base[a->n_apps];
  const bool cached = pairs && a->counts_build == a->build_serial;
  if (!a->last_plain) {
    // MAT store: per-node counts from k_digest, offsets scanned on the device (no host prefix,
    // no H2D of ptr); the fetch reuses the device offsets of the size query
    const size_t tw = scan_tmp_words(n);
    if (!cached) {
      gdroid_status st = ensure_scratch(a, (size_t)(n + 1 + tw) * 8);
      if (st) return st;
      CU(launch_scan_counts(a->D.node_popc, n, a->d_scratch, a->d_scratch + n + 1, a->stream));
      CU(cudaMemcpyAsync(ptr, a->d_scratch, (size_t)(n + 1) * 8, cudaMemcpyDeviceToHost, a->stream));
      CU(cudaStreamSynchronize(a->stream));
      a->counts_build = a->build_serial;
    }
    const uint64_t total = ptr[n];
    if (!pairs) return GDROID_OK;
    if (cap < total) return set_err(GDROID_E_SMALLBUF, "need %llu pairs, cap %llu", (unsigned long long)total, (unsigned long long)cap);
    gdroid_status st = ensure_scratch(a, (size_t)(n + 1 + tw) * 8 + (size_t)total * 8 + 8);
    if (st) return st;
    uint64_t* d_ptr = a->d_scratch;
    uint64_t* d_pairs = a->d_scratch + (n + 1 + tw);
    // the scratch may have been re-allocated (or used by another readback) since the size
    // query: rebuild the device offsets (a scan of the k_digest counts, ~1 ms per 16M nodes)
    CU(launch_scan_counts(a->D.node_popc, n, d_ptr, d_ptr + n + 1, a->stream));
    CU(launch_expand(a->D, 0, n, d_ptr, d_pairs, a->stream));
    CU(cudaMemcpyAsync(pairs, d_pairs, (size_t)total * 8, cudaMemcpyDeviceToHost, a->stream));
    CU(cudaStreamSynchronize(a->stream));
    return GDROID_OK;
  }
  if (!cached) {
    gdroid_status st = ensure_scratch(a, (size_t)(n + 1) * 8);
    if (st) return st;
    CU(launch_plain_sizes(a->P, 0, n, a->d_scratch, a->stream));
    CU(cudaMemcpyAsync(ptr + 1, a->d_scratch, (size_t)n * 8, cudaMemcpyDeviceToHost, a->stream));
    CU(cudaStreamSynchronize(a->stream));
    ptr[0] = 0;
    for (uint32_t i = 0; i < n; ++i) ptr[i + 1] += ptr[i];
    a->counts_build = a->build_serial;
  }
  const uint64_t total = ptr[n];
  if (!pairs) return GDROID_OK;
  if (cap < total) return set_err(GDROID_E_SMALLBUF, "need %llu pairs, cap %llu", (unsigned long long)total, (unsigned long long)cap);
  gdroid_status st = ensure_scratch(a, (size_t)(n + 1) * 8 + (size_t)total * 8 + 8);
  if (st) return st;
  uint64_t* d_ptr = a->d_scratch;
  uint64_t* d_pairs = a->d_scratch + (n + 1);
  CU(cudaMemcpyAsync(d_ptr, ptr, (size_t)(n + 1) * 8, cudaMemcpyHostToDevice, a->stream));
  CU(a->last_plain ? launch_plain_gather(a->P, 0, n, d_ptr, d_pairs, a->stream)
                   : launch_expand(a->D, 0, n, d_ptr, d_pairs, a->stream));
  CU(cudaMemcpyAsync(pairs, d_pairs, (size_t)total * 8, cudaMemcpyDeviceToHost, a->stream));
  CU(cudaStreamSynchronize(a->stream));
  return GDROID_OK;
}

// ---------------------------------------------------------------- incremental / out-of-core
gdroid_status gdroid_stage_seeds(gdroid_app* a, uint32_t k, uint32_t n, const uint32_t* nodes,
                                 const uint64_t* ptr, const uint64_t* pairs) {
  if (!a) return set_err(GDROID_E_INVALID, "app is NULL");
  if (k >= a->n_apps) return set_err(GDROID_E_RANGE, "app index %u >= %u", k, a->n_apps);
  if (n && (!nodes || !ptr)) return set_err(GDROID_E_INVALID, "nodes / ptr is NULL");
  const uint32_t n0 = a->app_base[k], nn = a->app_base[k + 1] - n0;
  for (uint32_t i = 0; i < n; ++i) {
    if (nodes[i] >= nn) return set_err(GDROID_E_RANGE, "seed %u: node %u >= %u", i, nodes[i], nn);
    if (ptr[i + 1] < ptr[i]) return set_err(GDROID_E_INVALID, "seed ptr not monotone at %u", i);
  }
  for (uint32_t i = 0; i < n; ++i) {
    a->seed_nodes.push_back(n0 + nodes[i]);
    for (uint64_t q = ptr[i]; q < ptr[i + 1]; ++q) {
      a->seed_pairs.push_back(n0 + nodes[i]);
      a->seed_pairs.push_back((uint32_t)(pairs[q] >> 32));
      a->seed_pairs.push_back((uint32_t)pairs[q]);
    }
  }
  return GDROID_OK;
}

// Facts of a list of nodes of app k (app-local ids) as CSR (ptr[n+1], pairs); two-call like
// gdroid_read_all_facts.  Used to read the boundary proxies of out-of-core sub-graphs.
gdroid_status gdroid_read_nodes_facts(const gdroid_app* ca, uint32_t k, uint32_t n, const uint32_t* nodes,
                                      uint64_t* ptr, uint64_t* pairs, uint64_t cap) {
  gdroid_app* a = const_cast<gdroid_app*>(ca);
  if (!a) return set_err(GDROID_E_INVALID, "app is NULL");
  if (!a->built) return set_err(GDROID_E_STATE, "facts read before a completed build");
  if (k >= a->n_apps) return set_err(GDROID_E_RANGE, "app index %u >= %u", k, a->n_apps);
  if (!ptr || (n && !nodes)) return set_err(GDROID_E_INVALID, "ptr / nodes is NULL");
  DeviceGuard guard(a->device);
  const uint32_t n0 = a->app_base[k], nn = a->app_base[k + 1] - n0;
  std::vector<uint32_t> gl(n);
  for (uint32_t i = 0; i < n; ++i) {
    if (nodes[i] >= nn) return set_err(GDROID_E_RANGE, "node %u >= %u", nodes[i], nn);
    gl[i] = n0 + nodes[i];
  }
  ptr[0] = 0;
  if (n == 0) return GDROID_OK;
  const size_t lw = (n + 1) / 2 + 1;                  // list words (u32 pairs) at the scratch start
  gdroid_status st = ensure_scratch(a, (lw + n + 1) * 8);
  if (st) return st;
  uint32_t* d_list = (uint32_t*)a->d_scratch;
  uint64_t* d_cnt = a->d_scratch + lw;
  CU(cudaMemcpyAsync(d_list, gl.data(), (size_t)n * 4, cudaMemcpyHostToDevice, a->stream));
  CU(launch_popc(a->D, 0, n, d_cnt, a->stream, d_list));
  CU(cudaMemcpyAsync(ptr + 1, d_cnt, (size_t)n * 8, cudaMemcpyDeviceToHost, a->stream));
  CU(cudaStreamSynchronize(a->stream));
  for (uint32_t i = 0; i < n; ++i) ptr[i + 1] += ptr[i];
  const uint64_t total = ptr[n];
  if (!pairs) return GDROID_OK;
  if (cap < total) return set_err(GDROID_E_SMALLBUF, "need %llu pairs, cap %llu", (unsigned long long)total, (unsigned long long)cap);
  st = ensure_scratch(a, (lw + n + 1 + total + 1) * 8);
  if (st) return st;
  d_list = (uint32_t*)a->d_scratch;
  d_cnt = a->d_scratch + lw;
  CU(cudaMemcpyAsync(d_list, gl.data(), (size_t)n * 4, cudaMemcpyHostToDevice, a->stream));
  CU(cudaMemcpyAsync(d_cnt, ptr, (size_t)(n + 1) * 8, cudaMemcpyHostToDevice, a->stream));
  CU(launch_expand(a->D, 0, n, d_cnt, d_cnt + n + 1, a->stream, d_list));
  CU(cudaMemcpyAsync(pairs, d_cnt + n + 1, (size_t)total * 8, cudaMemcpyDeviceToHost, a->stream));
  CU(cudaStreamSynchronize(a->stream));
  return GDROID_OK;
}

gdroid_status gdroid_read_reached(const gdroid_app* ca, uint32_t k, uint32_t n, const uint32_t* nodes, uint8_t* out) {
  gdroid_app* a = const_cast<gdroid_app*>(ca);
  if (!a) return set_err(GDROID_E_INVALID, "app is NULL");
  if (!a->digests_ok) return set_err(GDROID_E_STATE, "read before a completed build");
  if (k >= a->n_apps) return set_err(GDROID_E_RANGE, "app index %u >= %u", k, a->n_apps);
  DeviceGuard guard(a->device);
  const uint32_t n0 = a->app_base[k], nn = a->app_base[k + 1] - n0;
  std::vector<uint32_t> st(nn);
  CU(cudaMemcpyAsync(st.data(), a->D.stamp + n0, (size_t)nn * 4, cudaMemcpyDeviceToHost, a->stream));
  CU(cudaStreamSynchronize(a->stream));
  for (uint32_t i = 0; i < n; ++i) {
    if (nodes[i] >= nn) return set_err(GDROID_E_RANGE, "node %u >= %u", nodes[i], nn);
    out[i] = st[nodes[i]] != 0;
  }
  return GDROID_OK;
}

gdroid_status gdroid_export_facts(const gdroid_app* ca, void* host, uint64_t bytes) {
  gdroid_app* a = const_cast<gdroid_app*>(ca);
  if (!a) return set_err(GDROID_E_INVALID, "app is NULL");
  if (!a->d_facts || !a->facts_valid) return set_err(GDROID_E_STATE, "no facts to export");
  if (bytes != a->D.n_words * 8) return set_err(GDROID_E_SMALLBUF, "fact store is %llu B", (unsigned long long)(a->D.n_words * 8));
  if (a->pending) return set_err(GDROID_E_STATE, "an async build is still pending; call gdroid_sync");
  DeviceGuard guard(a->device);
  CU(cudaMemcpyAsync(host, a->d_facts, bytes, cudaMemcpyDeviceToHost, a->stream));
  return GDROID_OK;
}

gdroid_status gdroid_import_facts(gdroid_app* a, const void* host, uint64_t bytes) {
  if (!a) return set_err(GDROID_E_INVALID, "app is NULL");
  if (bytes != a->D.n_words * 8) return set_err(GDROID_E_SMALLBUF, "fact store is %llu B", (unsigned long long)(a->D.n_words * 8));
  if (a->pending) return set_err(GDROID_E_STATE, "an async build is still pending; call gdroid_sync");
  DeviceGuard guard(a->device);
  gdroid_status st = ensure_facts(a);
  if (st) return st;
  CU(cudaMemcpyAsync(a->d_facts, host, bytes, cudaMemcpyHostToDevice, a->stream));
  a->facts_valid = true;
  a->mask_stale = true;                               // narrow masks are rebuilt by the next keep build
  a->built = false;                                   // facts no longer those of a build
  return GDROID_OK;
}

gdroid_status gdroid_stream_sync(gdroid_app* a) {
  if (!a) return set_err(GDROID_E_INVALID, "app is NULL");
  DeviceGuard guard(a->device);
  CU(cudaStreamSynchronize(a->stream));
  return GDROID_OK;
}

uint64_t gdroid_fact_bytes(const gdroid_app* a) { return a ? a->D.n_words * 8 : 0; }

// Asynchronous whole-batch readback: offsets scanned on the device (one small
// synchronous copy of the pair count), pairs expanded on the device, then ptr (n+1 words) and
// the pairs copied to the caller's PINNED buffers by the copy engine without waiting — the copy
// overlaps whatever the caller enqueues next (the next batch's fixed point).  Complete with
// gdroid_stream_sync.  *total gets the pair count; GDROID_E_SMALLBUF (nothing copied) if it
// exceeds cap.
gdroid_status gdroid_read_batch_facts_async(gdroid_app* a, uint64_t* ptr, uint64_t* pairs, uint64_t cap,
                                            uint64_t* total, uint32_t blocks) {
  (void)blocks;
  if (!a) return set_err(GDROID_E_INVALID, "app is NULL");
  if (!a->built || a->last_plain) return set_err(GDROID_E_STATE, "async readback needs a completed MAT build with facts");
  if (!ptr || !pairs || !total) return set_err(GDROID_E_INVALID, "ptr / pairs / total is NULL");
  DeviceGuard guard(a->device);
  const uint32_t n = a->app_base[a->n_apps];
  const size_t tw = scan_tmp_words(n);
  gdroid_status st = ensure_scratch(a, (size_t)(n + 1 + tw) * 8);
  if (st) return st;
  CU(launch_scan_counts(a->D.node_popc, n, a->d_scratch, a->d_scratch + n + 1, a->stream));
  CU(cudaMemcpyAsync(total, a->d_scratch + n, 8, cudaMemcpyDeviceToHost, a->stream));
  CU(cudaStreamSynchronize(a->stream));
  const uint64_t tot = *total;
  if (tot > cap) return set_err(GDROID_E_SMALLBUF, "need %llu pairs, cap %llu", (unsigned long long)tot, (unsigned long long)cap);
  const size_t need = (size_t)(n + 1 + tw) * 8 + (size_t)tot * 8 + 8;
  if (a->scratch_bytes < need) {                     // grown: the offsets move with the scratch
    st = ensure_scratch(a, need);
    if (st) return st;
    CU(launch_scan_counts(a->D.node_popc, n, a->d_scratch, a->d_scratch + n + 1, a->stream));
  }
  uint64_t* d_ptr = a->d_scratch;
  uint64_t* d_pairs = a->d_scratch + (n + 1 + tw);
  CU(launch_expand(a->D, 0, n, d_ptr, d_pairs, a->stream));
  CU(cudaMemcpyAsync(ptr, d_ptr, (size_t)(n + 1) * 8, cudaMemcpyDeviceToHost, a->stream));
  CU(cudaMemcpyAsync(pairs, d_pairs, (size_t)tot * 8, cudaMemcpyDeviceToHost, a->stream));
  a->counts_build = ~0ull;                            // scratch now holds pairs after the offsets
  return GDROID_OK;
}

gdroid_status gdroid_release_facts(gdroid_app* a) {
  if (!a) return set_err(GDROID_E_INVALID, "app is NULL");
  if (a->pending) return set_err(GDROID_E_STATE, "an async build is still pending; call gdroid_sync");
  if (!a->d_facts) return GDROID_OK;
  DeviceGuard guard(a->device);
  facts_free(a->device, a->d_facts, a->fact_block_bytes, a->stream);
  a->d_facts = nullptr;
  a->D.facts = a->D.delta = nullptr;
  a->facts_valid = false;
  a->built = false;                                   // digests stay readable
  return GDROID_OK;
}

uint32_t gdroid_n_apps(const gdroid_app* a) { return a ? a->n_apps : 0; }

gdroid_status gdroid_read_all_facts(const gdroid_app* ca, uint32_t k, uint64_t* ptr, uint64_t* pairs, uint64_t cap) {
  gdroid_app* a = const_cast<gdroid_app*>(ca);
  if (!a) return set_err(GDROID_E_INVALID, "app is NULL");
  if (!a->built) return set_err(GDROID_E_STATE, "facts read before a completed build");
  if (k >= a->n_apps) return set_err(GDROID_E_RANGE, "app index %u >= %u", k, a->n_apps);
  if (!ptr) return set_err(GDROID_E_INVALID, "ptr is NULL");
  DeviceGuard guard(a->device);
  const uint32_t n0 = a->app_base[k], n1 = a->app_base[k + 1], n = n1 - n0;
  gdroid_status st = ensure_scratch(a, (size_t)(n + 1) * 8);
  if (st) return st;
  CU(a->last_plain ? launch_plain_sizes(a->P, n0, n1, a->d_scratch, a->stream)
                   : launch_popc(a->D, n0, n1, a->d_scratch, a->stream));
  std::vector<uint64_t> cnt(n);
  CU(cudaMemcpyAsync(cnt.data(), a->d_scratch, (size_t)n * 8, cudaMemcpyDeviceToHost, a->stream));
  CU(cudaStreamSynchronize(a->stream));
  ptr[0] = 0;
  for (uint32_t i = 0; i < n; ++i) ptr[i + 1] = ptr[i] + cnt[i];
  const uint64_t total = ptr[n];
  if (!pairs) return GDROID_OK;
  if (cap < total) return set_err(GDROID_E_SMALLBUF, "need %llu pairs, cap %llu", (unsigned long long)total, (unsigned long long)cap);
  st = ensure_scratch(a, (size_t)(n + 1) * 8 + (size_t)total * 8 + 8);
  if (st) return st;
  uint64_t* d_ptr = a->d_scratch;
  uint64_t* d_pairs = a->d_scratch + (n + 1);
  CU(cudaMemcpyAsync(d_ptr, ptr, (size_t)(n + 1) * 8, cudaMemcpyHostToDevice, a->stream));
  CU(a->last_plain ? launch_plain_gather(a->P, n0, n1, d_ptr, d_pairs, a->stream)
                   : launch_expand(a->D, n0, n1, d_ptr, d_pairs, a->stream));
  CU(cudaMemcpyAsync(pairs, d_pairs, (size_t)total * 8, cudaMemcpyDeviceToHost, a->stream));
  CU(cudaStreamSynchronize(a->stream));
  return GDROID_OK;
}

gdroid_status gdroid_read_facts_in(const gdroid_app* ca, uint32_t k, uint32_t node, uint64_t* pairs, uint64_t cap,
                                   uint64_t* n_pairs) {
  gdroid_app* a = const_cast<gdroid_app*>(ca);
  if (!a) return set_err(GDROID_E_INVALID, "app is NULL");
  if (!a->built) return set_err(GDROID_E_STATE, "facts read before a completed build");
  if (k >= a->n_apps) return set_err(GDROID_E_RANGE, "app index %u >= %u", k, a->n_apps);
  const uint32_t n0 = a->app_base[k], n1 = a->app_base[k + 1];
  if (node >= n1 - n0) return set_err(GDROID_E_RANGE, "node %u >= n_nodes %u", node, n1 - n0);
  if (!n_pairs) return set_err(GDROID_E_INVALID, "n_pairs is NULL");
  DeviceGuard guard(a->device);
  gdroid_status st = ensure_scratch(a, 16);
  if (st) return st;
  const uint32_t g = n0 + node;
  CU(a->last_plain ? launch_plain_sizes(a->P, g, g + 1, a->d_scratch, a->stream)
                   : launch_popc(a->D, g, g + 1, a->d_scratch, a->stream));
  uint64_t cnt = 0;
  CU(cudaMemcpyAsync(&cnt, a->d_scratch, 8, cudaMemcpyDeviceToHost, a->stream));
  CU(cudaStreamSynchronize(a->stream));
  *n_pairs = cnt;
  if (!pairs) return GDROID_OK;
  if (cap < cnt) return set_err(GDROID_E_SMALLBUF, "need %llu pairs, cap %llu", (unsigned long long)cnt, (unsigned long long)cap);
  st = ensure_scratch(a, 16 + (size_t)cnt * 8);
  if (st) return st;
  uint64_t zero = 0;
  CU(cudaMemcpyAsync(a->d_scratch, &zero, 8, cudaMemcpyHostToDevice, a->stream));
  CU(a->last_plain ? launch_plain_gather(a->P, g, g + 1, a->d_scratch, a->d_scratch + 2, a->stream)
                   : launch_expand(a->D, g, g + 1, a->d_scratch, a->d_scratch + 2, a->stream));
  CU(cudaMemcpyAsync(pairs, a->d_scratch + 2, (size_t)cnt * 8, cudaMemcpyDeviceToHost, a->stream));
  CU(cudaStreamSynchronize(a->stream));
  return GDROID_OK;
}

gdroid_status gdroid_read_facts(const gdroid_app* a, uint32_t node, uint64_t* pairs, uint64_t cap, uint64_t* n_pairs) {
  return gdroid_read_facts_in(a, 0, node, pairs, cap, n_pairs);
}

gdroid_status gdroid_node_digests_in(const gdroid_app* ca, uint32_t k, uint64_t* per_node, uint64_t* app_digest) {
  gdroid_app* a = const_cast<gdroid_app*>(ca);
  if (!a) return set_err(GDROID_E_INVALID, "app is NULL");
  if (!a->digests_ok) return set_err(GDROID_E_STATE, "digests read before a completed build");
  if (k >= a->n_apps) return set_err(GDROID_E_RANGE, "app index %u >= %u", k, a->n_apps);
  DeviceGuard guard(a->device);
  const uint32_t n0 = a->app_base[k], n = a->app_base[k + 1] - n0;
  if (per_node) CU(cudaMemcpyAsync(per_node, a->D.node_digest + n0, (size_t)n * 8, cudaMemcpyDeviceToHost, a->stream));
  if (app_digest) CU(cudaMemcpyAsync(app_digest, a->D.app_digest + k, 8, cudaMemcpyDeviceToHost, a->stream));
  CU(cudaStreamSynchronize(a->stream));
  return GDROID_OK;
}

gdroid_status gdroid_node_digests(const gdroid_app* a, uint64_t* per_node, uint64_t* app_digest) {
  return gdroid_node_digests_in(a, 0, per_node, app_digest);
}

gdroid_status gdroid_app_digests(const gdroid_app* ca, uint64_t* per_app) {
  gdroid_app* a = const_cast<gdroid_app*>(ca);
  if (!a || !per_app) return set_err(GDROID_E_INVALID, "NULL argument");
  if (!a->digests_ok) return set_err(GDROID_E_STATE, "digests read before a completed build");
  DeviceGuard guard(a->device);
  CU(cudaMemcpyAsync(per_app, a->D.app_digest, (size_t)a->n_apps * 8, cudaMemcpyDeviceToHost, a->stream));
  CU(cudaStreamSynchronize(a->stream));
  return GDROID_OK;
}

void gdroid_free(gdroid_app* a) { free_app(a); }

gdroid_status gdroid_debug_phases(const gdroid_app* a, uint64_t* out8) {
  if (!a || !out8) return set_err(GDROID_E_INVALID, "NULL argument");
  for (int i = 0; i < 8; ++i) out8[i] = a->h_stats->phase[i];
  return GDROID_OK;
}

gdroid_status gdroid_debug_tables(const gdroid_app* a, uint32_t which, void* host, uint64_t cap, uint64_t* bytes) {
  if (!a || !bytes) return set_err(GDROID_E_INVALID, "NULL argument");
  if (which > 8) return set_err(GDROID_E_RANGE, "table %u", which);
  const Dev& D = a->D;
  const void* src[9] = {D.nodes, D.edges, D.inl, D.frow, D.xmap, D.args, D.row_ptr, D.arg_ptr, D.node_method};
  const uint64_t esz[9] = {sizeof(NodeRec), sizeof(Edge), sizeof(InlEdge), 4, 4, 4, 4, 4, 4};
  *bytes = a->tab_len[which] * esz[which];
  if (!host) return GDROID_OK;
  if (cap < *bytes) return set_err(GDROID_E_SMALLBUF, "need %llu bytes", (unsigned long long)*bytes);
  DeviceGuard guard(a->device);
  CU(cudaStreamSynchronize(a->stream));
  if (*bytes) CU(cudaMemcpy(host, src[which], *bytes, cudaMemcpyDeviceToHost));
  return GDROID_OK;
}

gdroid_status gdroid_debug_trace(gdroid_app* a, uint32_t cap) {
  if (!a) return set_err(GDROID_E_INVALID, "app is NULL");
  DeviceGuard guard(a->device);
  if (a->D.trace) { cudaFree(a->D.trace); a->D.trace = nullptr; }
  a->D.trace_cap = 0;
  if (cap) {
    CU(cudaMalloc(&a->D.trace, (size_t)cap * 16));
    CU(cudaMemset(a->D.trace, 0, (size_t)cap * 16));
    a->D.trace_cap = cap;
  }
  return GDROID_OK;
}

gdroid_status gdroid_debug_read_trace(const gdroid_app* ca, uint64_t* out, uint64_t cap, uint64_t* n) {
  gdroid_app* a = const_cast<gdroid_app*>(ca);
  if (!a || !n) return set_err(GDROID_E_INVALID, "NULL argument");
  if (!a->built) return set_err(GDROID_E_STATE, "trace read before a completed build");
  DeviceGuard guard(a->device);
  const uint64_t r = std::min<uint64_t>(a->last.rounds + 1, a->D.trace_cap);
  *n = r;
  if (!out) return GDROID_OK;
  if (cap < 2 * r) return set_err(GDROID_E_SMALLBUF, "need %llu words", (unsigned long long)(2 * r));
  CU(cudaMemcpy(out, a->D.trace, r * 16, cudaMemcpyDeviceToHost));
  return GDROID_OK;
}

}  // extern "C"
