// plain.cu — the set-based PLAIN variant of the ablation.
//
// Alg. 2 "Kernel of Plain GPU Implementation", recast on B200 as a
// persistent cooperative kernel with one device round per worklist:
//   * one THREAD per worklist node (Alg. 2 l.5, l.10-11: "one thread processes one node");
//   * the node's GEN_KILL is a per-thread switch over the node kinds (l.12; the 25-way branch
//     the paper blames for divergence);
//   * fact sets are the set-based structure of Fig. 5a: every node owns a
//     sorted array of (slot gid << 32 | instance gid) pairs in a device heap; a union that
//     outgrows the array re-allocates it from a bump allocator and copies (the dynamic
//     allocation of PAPER.md:667-691; the old array is not reused);
//   * SEARCH + union + update() (l.13-17): per out-edge the edge transform, then a sorted
//     merge into the destination's array under the destination's lock; a destination that
//     grew (or was never reached, DESIGN.md §3 A5) is inserted into the next worklist (a set:
//     round-stamp test-and-set).
// Same least fixed point as the MAT path; only the data structure and the mapping differ.
#include "internal.cuh"

namespace gd {
namespace {

constexpr uint64_t NONE = ~0ull;

__device__ __forceinline__ uint32_t slot_of(uint64_t p) { return (uint32_t)(p >> 32); }
__device__ __forceinline__ uint64_t pack(uint64_t s, uint64_t o) { return (s << 32) | o; }

// first index i in [lo, hi) with a[i] >= key (a sorted, read through L2)
__device__ uint64_t lower_bound64(const uint64_t* a, uint64_t lo, uint64_t hi, uint64_t key) {
  while (lo < hi) {
    const uint64_t mid = (lo + hi) >> 1;
    if (__ldcg(a + mid) < key) lo = mid + 1; else hi = mid;
  }
  return lo;
}
template <class T>
__device__ bool contains_sorted(const T* a, uint64_t lo, uint64_t hi, T key) {
  while (lo < hi) {
    const uint64_t mid = (lo + hi) >> 1;
    const T v = a[mid];
    if (v == key) return true;
    if (v < key) lo = mid + 1; else hi = mid;
  }
  return false;
}

// Instances o with (s, o) in X[0, n): the index range [*b, *e).
__device__ __forceinline__ void pts(const uint64_t* X, uint64_t n, int64_t s, uint64_t* b, uint64_t* e) {
  if (s < 0) { *b = *e = 0; return; }
  *b = lower_bound64(X, 0, n, pack((uint64_t)s, 0));
  *e = lower_bound64(X, *b, n, pack((uint64_t)s + 1, 0));
}

// heap slot gid of (o, f): o != NULL and f in F(t(o)) (DESIGN.md §3 C1), else -1
__device__ int64_t heap_slot(const PlainDev& P, uint32_t o, uint32_t f) {
  if (o == 0) return -1;
  const int32_t t = P.inst_type[o];
  if (t < 0) return -1;
  uint64_t lo = P.tf_ptr[t], hi = P.tf_ptr[t + 1];
  const uint64_t base = lo;
  while (lo < hi) {
    const uint64_t mid = (lo + hi) >> 1;
    const uint32_t v = P.tfields[mid];
    if (v == f) return (int64_t)(P.L_total + P.G + P.heap_base[o] + (mid - base));
    if (v < f) lo = mid + 1; else hi = mid;
  }
  return -1;
}

// pool membership of module d (π, DESIGN.md §3 C1): instance o in Q_d; global slot s in P_d
__device__ __forceinline__ bool in_Q(const PlainDev& P, uint32_t d, uint32_t o) {
  return contains_sorted(P.insts, P.inst_ptr[d], P.inst_ptr[d + 1], o);
}
__device__ bool in_P_global(const PlainDev& P, uint32_t d, uint64_t s) {
  if (s < P.L_total + P.G) return contains_sorted(P.statics, P.stat_ptr[d], P.stat_ptr[d + 1], (uint32_t)(s - P.L_total));
  const uint64_t h = s - P.L_total - P.G;            // owner: last o with heap_base[o] <= h
  uint64_t lo = 0, hi = P.n_instances;
  while (lo + 1 < hi) {
    const uint64_t mid = (lo + hi) >> 1;
    if (P.heap_base[mid] <= h) lo = mid; else hi = mid;
  }
  return in_Q(P, d, (uint32_t)lo);
}

// Z = (X without the pairs of slot `kill`) ∪ G, X and G sorted; returns |Z|
__device__ uint64_t merge_kill(const uint64_t* X, uint64_t nx, int64_t kill, const uint64_t* G, uint64_t ng,
                               uint64_t* Z) {
  uint64_t i = 0, j = 0, k = 0;
  while (i < nx || j < ng) {
    if (i < nx && kill >= 0 && slot_of(X[i]) == (uint32_t)kill) { ++i; continue; }
    uint64_t v;
    if (j >= ng || (i < nx && X[i] < G[j])) v = X[i++];
    else if (i >= nx || G[j] < X[i]) v = G[j++];
    else { v = X[i]; ++i; ++j; }
    Z[k++] = v;
  }
  return k;
}

// shell sort + unique (FLOAD's generated pairs come as several sorted runs)
__device__ uint64_t sort_unique(uint64_t* a, uint64_t n) {
  for (uint64_t gap = n / 2; gap > 0; gap /= 2)
    for (uint64_t i = gap; i < n; ++i) {
      const uint64_t v = a[i];
      uint64_t j = i;
      for (; j >= gap && a[j - gap] > v; j -= gap) a[j] = a[j - gap];
      a[j] = v;
    }
  uint64_t k = 0;
  for (uint64_t i = 0; i < n; ++i)
    if (k == 0 || a[k - 1] != a[i]) a[k++] = a[i];
  return k;
}

// GEN_KILL of node n (DESIGN.md §3 C2): Y = f(X); C is scratch.  Returns |Y|.
__device__ uint64_t transfer(const PlainDev& P, uint32_t n, const uint64_t* X, uint64_t nx, uint64_t* Y,
                             uint64_t* C) {
  const int32_t* op = P.ops + 4ull * n;
  const uint32_t m = P.nmeth[n];
  uint64_t b, e, nc = 0;
  switch (P.nkind[n]) {
    case GK_PRIM:
      return merge_kill(X, nx, op[0], C, 0, Y);
    case GK_CONST: case GK_NEW:
      if (op[0] < 0) return merge_kill(X, nx, -1, C, 0, Y);
      C[0] = pack((uint64_t)op[0], (uint32_t)op[3]);
      return merge_kill(X, nx, op[0], C, 1, Y);
    case GK_COPY: case GK_SLOAD: case GK_SSTORE: case GK_RETV: {
      const int64_t v = (P.nkind[n] == GK_RETV) ? (int64_t)(P.local_base[m + 1] - 1) : (int64_t)op[0];
      pts(X, nx, op[1], &b, &e);
      if (v >= 0)
        for (uint64_t i = b; i < e; ++i) C[nc++] = pack((uint64_t)v, (uint32_t)X[i]);
      return merge_kill(X, nx, P.nkind[n] == GK_SSTORE ? -1 : v, C, nc, Y);   // SSTORE: weak
    }
    case GK_FLOAD: case GK_ALOAD: {                                            // v = w.f
      const uint32_t f = P.nkind[n] == GK_ALOAD ? GDROID_F_ARR : (uint32_t)op[2];
      pts(X, nx, op[1], &b, &e);
      for (uint64_t i = b; i < e && op[0] >= 0; ++i) {
        const int64_t hs = heap_slot(P, (uint32_t)X[i], f);
        if (hs < 0) continue;                                                  // NULL: no fields
        uint64_t b2, e2;
        pts(X, nx, hs, &b2, &e2);
        for (uint64_t q = b2; q < e2; ++q) {
          if (nc == P.maxset) nc = sort_unique(C, nc);
          C[nc++] = pack((uint64_t)op[0], (uint32_t)X[q]);
        }
      }
      nc = sort_unique(C, nc);
      return merge_kill(X, nx, op[0], C, nc, Y);
    }
    case GK_FSTORE: case GK_ASTORE: {                                          // v.f = w (weak)
      const uint32_t f = P.nkind[n] == GK_ASTORE ? GDROID_F_ARR : (uint32_t)op[2];
      uint64_t bw, ew;
      pts(X, nx, op[0], &b, &e);
      pts(X, nx, op[1], &bw, &ew);
      for (uint64_t i = b; i < e; ++i) {                  // o1 ascending -> heap slots ascending
        const int64_t hs = heap_slot(P, (uint32_t)X[i], f);
        if (hs < 0) continue;
        for (uint64_t q = bw; q < ew; ++q) C[nc++] = pack((uint64_t)hs, (uint32_t)X[q]);
      }
      return merge_kill(X, nx, -1, C, nc, Y);
    }
    default:                                                                   // identity kinds
      for (uint64_t i = 0; i < nx; ++i) Y[i] = X[i];
      return nx;
  }
}

// Edge transform T_e (DESIGN.md §3 C3) of Y along p -> s into Z (sorted); returns |Z|.
__device__ uint64_t edge_transform(const PlainDev& P, uint32_t p, uint32_t s, uint32_t kind, const uint64_t* Y,
                                   uint64_t ny, uint64_t* Z) {
  uint64_t nz = 0, b, e;
  const uint64_t g0 = lower_bound64(Y, 0, ny, pack(P.L_total, 0));          // first global pair
  if (kind == GE_C2R) {                                                      // locals except lhs(c)
    const uint32_t m = P.nmeth[p];
    const int32_t lhs = P.ops[4ull * p];
    for (uint64_t i = 0; i < g0; ++i) {
      const uint64_t sl = slot_of(Y[i]);
      if (sl >= P.local_base[m] && sl < P.local_base[m + 1] && (int64_t)sl != lhs) Z[nz++] = Y[i];
    }
    for (uint64_t i = g0; i < ny; ++i) Z[nz++] = Y[i];
    return nz;
  }
  const uint32_t mt = P.nmeth[s], d = P.mmod[mt];
  if (kind == GE_CALL) {                                                     // params <- args
    const uint32_t np = P.n_params[mt];
    for (uint32_t j = 0; j < np; ++j) {
      const int32_t a = P.args[P.arg_ptr[p] + j];
      pts(Y, ny, a, &b, &e);
      for (uint64_t i = b; i < e; ++i)
        if (in_Q(P, d, (uint32_t)Y[i])) Z[nz++] = pack(P.local_base[mt] + j, (uint32_t)Y[i]);
    }
  } else {                                                                   // GE_RET: lhs(c) <- RET
    const int32_t lhs = P.ops[4ull * s];                                     // RETSITE op0 = lhs(c)
    const uint32_t mc = P.nmeth[p];
    if (lhs >= 0) {
      pts(Y, ny, (int64_t)(P.local_base[mc + 1] - 1), &b, &e);
      for (uint64_t i = b; i < e; ++i)
        if (in_Q(P, d, (uint32_t)Y[i])) Z[nz++] = pack((uint64_t)lhs, (uint32_t)Y[i]);
    }
  }
  for (uint64_t i = g0; i < ny; ++i)                                         // Glob(Y) ∩ π
    if (in_P_global(P, d, slot_of(Y[i])) && in_Q(P, d, (uint32_t)Y[i])) Z[nz++] = Y[i];
  return nz;
}

__device__ __forceinline__ void lock(uint32_t* l) {
  while (atomicCAS(l, 0u, 1u) != 0u) __nanosleep(32);
  __threadfence();
}
__device__ __forceinline__ void unlock(uint32_t* l) {
  __threadfence();
  atomicExch(l, 0u);
}

// IN(s) ∪= T under s's lock; regrows the array from the bump allocator.  Returns grew.
__device__ bool union_into(const PlainDev& P, uint32_t s, const uint64_t* T, uint64_t nt, unsigned long long& allocs) {
  if (nt == 0) return false;
  lock(&P.locks[s]);
  SetDesc d;
  d.off = __ldcg(&P.sets[s].off);
  d.size = __ldcg(&P.sets[s].size);
  d.cap = __ldcg(&P.sets[s].cap);
  const uint64_t* H = P.heap + d.off;
  uint64_t i = 0, j = 0, fresh = 0;
  while (j < nt) {                                                           // count new pairs
    const uint64_t h = i < d.size ? __ldcg(H + i) : NONE;
    if (i < d.size && h < T[j]) ++i;
    else if (i < d.size && h == T[j]) { ++i; ++j; }
    else { ++fresh; ++j; }
  }
  if (fresh == 0) { unlock(&P.locks[s]); return false; }
  const uint64_t need = d.size + fresh;
  if (need > d.cap) {                                                        // re-allocate + merge
    uint64_t ncap = d.cap * 2 > need ? d.cap * 2 : need;
    if (ncap < 8) ncap = 8;
    const unsigned long long off = atomicAdd(P.heap_top, (unsigned long long)ncap);
    if (off + ncap > P.heap_cap) { atomicExch(P.err, 1u); unlock(&P.locks[s]); return false; }
    ++allocs;
    uint64_t* Z = P.heap + off;
    i = 0; j = 0;
    uint64_t k = 0;
    while (i < d.size || j < nt) {
      const uint64_t h = i < d.size ? __ldcg(H + i) : NONE;
      if (j >= nt || (i < d.size && h < T[j])) { Z[k++] = h; ++i; }
      else if (i >= d.size || T[j] < h) Z[k++] = T[j++];
      else { Z[k++] = h; ++i; ++j; }
    }
    d.off = off;
    d.cap = (uint32_t)ncap;
  } else {                                                                   // in place, from the back
    uint64_t* Z = P.heap + d.off;
    int64_t a = (int64_t)d.size - 1, bb = (int64_t)nt - 1, w = (int64_t)need - 1;
    while (bb >= 0) {
      const uint64_t h = a >= 0 ? __ldcg(Z + a) : 0;
      if (a >= 0 && h > T[bb]) { Z[w--] = h; --a; }
      else if (a >= 0 && h == T[bb]) { Z[w--] = h; --a; --bb; }
      else Z[w--] = T[bb--];
    }
  }
  d.size = (uint32_t)need;
  P.sets[s] = d;
  unlock(&P.locks[s]);
  return true;
}

// ---- CELL variant: the cell-major per-method matrix store (Fig. 5b)
// row of slot gid `sl` in method m's matrix (locals first, then the module's global rows)
__device__ int64_t cell_row(const PlainDev& P, uint32_t m, uint64_t sl) {
  if (sl >= P.local_base[m] && sl < P.local_base[m + 1]) return (int64_t)(sl - P.local_base[m]);
  const uint32_t d = P.mmod[m];
  uint32_t lo = P.mgrow_ptr[d], hi = P.mgrow_ptr[d + 1];
  const uint32_t base = lo;
  while (lo < hi) {
    const uint32_t mid = (lo + hi) >> 1;
    if (P.mgrow[mid] < sl) lo = mid + 1; else hi = mid;
  }
  if (lo < P.mgrow_ptr[d + 1] && P.mgrow[lo] == sl) return (int64_t)(P.local_base[m + 1] - P.local_base[m]) + (lo - base);
  return -1;
}
__device__ int64_t cell_col(const PlainDev& P, uint32_t m, uint32_t o) {
  const uint32_t d = P.mmod[m];
  uint64_t lo = P.inst_ptr[d], hi = P.inst_ptr[d + 1];
  const uint64_t base = lo;
  while (lo < hi) {
    const uint64_t mid = (lo + hi) >> 1;
    if (P.insts[mid] < o) lo = mid + 1; else hi = mid;
  }
  return (lo < P.inst_ptr[d + 1] && P.insts[lo] == o) ? (int64_t)(lo - base) : -1;
}

// IN(n) from the cell store: bit nidx(n) of every cell of its method's matrix, row-major =
// ascending (slot gid, instance gid).  Read through L2 (cells are OR-ed by other threads).
__device__ uint64_t cell_gather(const PlainDev& P, uint32_t n, uint64_t* A) {
  const uint32_t m = P.nmeth[n], d = P.mmod[m];
  const uint32_t rows = P.m_rows[m], cols = P.m_cols[m], wpc = P.m_wpc[m], i = P.nidx[n];
  const uint64_t* C = P.cells + P.m_coff[m] + (i >> 6);
  const uint64_t bit = 1ull << (i & 63);
  const uint32_t nloc = (uint32_t)(P.local_base[m + 1] - P.local_base[m]);
  uint64_t k = 0;
  for (uint32_t r = 0; r < rows; ++r) {
    const uint64_t sl = r < nloc ? P.local_base[m] + r : P.mgrow[P.mgrow_ptr[d] + (r - nloc)];
    for (uint32_t c = 0; c < cols; ++c)
      if (__ldcg(C + ((uint64_t)r * cols + c) * wpc) & bit) A[k++] = pack(sl, P.insts[P.inst_ptr[d] + c]);
  }
  return k;
}

// IN(s) ∪= T on the cell store: one atomicOr of bit nidx(s) per pair; grew = some bit was new.
__device__ bool cell_union(const PlainDev& P, uint32_t s, const uint64_t* T, uint64_t nt) {
  const uint32_t m = P.nmeth[s], cols = P.m_cols[m], wpc = P.m_wpc[m], i = P.nidx[s];
  uint64_t* C = P.cells + P.m_coff[m] + (i >> 6);
  const uint64_t bit = 1ull << (i & 63);
  bool grew = false;
  for (uint64_t j = 0; j < nt; ++j) {
    const int64_t r = cell_row(P, m, slot_of(T[j])), c = cell_col(P, m, (uint32_t)T[j]);
    if (r < 0 || c < 0) { atomicExch(P.err, 2u); continue; }           // outside P_m x Q_m (never: π)
    unsigned long long* w = (unsigned long long*)(C + ((uint64_t)r * cols + (uint64_t)c) * wpc);
    if (__ldcg((const uint64_t*)w) & bit) continue;                     // (IN only grows)
    if (!(atomicOr(w, bit) & bit)) grew = true;
  }
  return grew;
}

__device__ __forceinline__ void push(const PlainDev& P, uint32_t s, uint32_t round) {
  if (atomicMax(&P.stamp[s], round + 1) < round + 1) {                      // set insert (dedupe)
    const uint32_t q = (round + 1) % 3;
    const uint32_t idx = atomicAdd(&P.counts[q], 1u);
    P.queue[(size_t)q * P.n_nodes + idx] = s;
  }
}

__device__ __forceinline__ void plain_grid_sync(uint32_t* bar, uint32_t nblocks) {
  __syncthreads();
  if (threadIdx.x == 0) {
    volatile uint32_t* vgen = bar + 1;
    const uint32_t gen = *vgen;
    __threadfence();
    if (atomicAdd(bar, 1u) == nblocks - 1) {
      atomicExch(bar, 0u);
      __threadfence();
      atomicAdd(bar + 1, 1u);
    } else {
      while (*vgen == gen) __nanosleep(20);
    }
    __threadfence();
  }
  __syncthreads();
}

__global__ void k_plain_seed(PlainDev P) {
  for (uint32_t i = threadIdx.x; i < P.n_entries; i += blockDim.x) push(P, P.entries[i], 0u);
}

__global__ void __launch_bounds__(128) k_plain_fixpoint(PlainDev P) {
  const uint64_t tid = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
  const uint64_t nth = (uint64_t)gridDim.x * blockDim.x;
  uint64_t* A = P.scratch + tid * 3 * P.maxset;
  uint64_t* B = A + P.maxset;
  uint64_t* C = B + P.maxset;
  unsigned long long visits = 0, allocs = 0;
  for (uint32_t round = 1;; ++round) {
    const uint32_t cur = round % 3;
    const uint32_t total = __ldcg(&P.counts[cur]);
    if (total == 0) break;                                                   // Alg. 2 l.8
    if (P.max_rounds && round > P.max_rounds) {
      if (tid == 0) P.stats->limit_hit = 1;
      break;
    }
    if (tid == 0) {
      P.counts[(round + 2) % 3] = 0;
      P.stats->rounds += 1;
      P.stats->hist[total <= 32 ? 0 : (total <= 64 ? 1 : 2)] += 1;
    }
    for (uint64_t it = tid; it < total; it += nth) {                         // l.9-11: thread per node
      const uint32_t n = __ldcg(&P.queue[(size_t)cur * P.n_nodes + it]);
      ++visits;
      uint64_t sz;
      if (P.cell) {
        sz = cell_gather(P, n, A);                                           // IN(n) from the cells
      } else {
        lock(&P.locks[n]);                                                   // snapshot of IN(n)
        const uint64_t off = __ldcg(&P.sets[n].off);
        sz = __ldcg(&P.sets[n].size);
        for (uint32_t i = 0; i < sz; ++i) A[i] = __ldcg(P.heap + off + i);
        unlock(&P.locks[n]);
      }
      const uint64_t ny = transfer(P, n, A, sz, B, C);                      // l.12 GEN_KILL
      for (uint64_t e = P.row_ptr[n]; e < P.row_ptr[n + 1]; ++e) {          // l.13-17
        const uint32_t s = P.col[e], k = P.ekind[e];
        const uint64_t* T = B;
        uint64_t nt = ny;
        if (k != GE_INTRA) { nt = edge_transform(P, n, s, k, B, ny, C); T = C; }
        const bool grew = P.cell ? cell_union(P, s, T, nt) : union_into(P, s, T, nt, allocs);
        if (grew || __ldcg(&P.stamp[s]) == 0) push(P, s, round);
      }
    }
    plain_grid_sync(P.bar, gridDim.x);                                       // l.18 syncthread
  }
  if (visits) atomicAdd(&P.stats->visits, visits);
  if (allocs) atomicAdd(&P.stats->atomics, allocs);                          // (re)allocations
}

// per-node sizes (readback) and gather into CSR order
__global__ void k_plain_sizes(PlainDev P, uint32_t n0, uint32_t n1, uint64_t* out) {
  for (uint32_t n = n0 + blockIdx.x * blockDim.x + threadIdx.x; n < n1; n += gridDim.x * blockDim.x)
    out[n - n0] = P.sets[n].size;
}
__global__ void k_plain_gather(PlainDev P, uint32_t n0, uint32_t n1, const uint64_t* ptr, uint64_t* pairs) {
  const int lane = threadIdx.x & 31;
  const uint32_t nw = gridDim.x * (blockDim.x >> 5);
  for (uint32_t n = n0 + blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); n < n1; n += nw) {
    const SetDesc d = P.sets[n];
    for (uint32_t i = lane; i < d.size; i += 32) pairs[ptr[n - n0] + i] = P.heap[d.off + i];
  }
}

__device__ __forceinline__ uint64_t mix64p(uint64_t z) {   // splitmix64 finaliser (C8)
  z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ULL;
  z = (z ^ (z >> 27)) * 0x94d049bb133111ebULL;
  return z ^ (z >> 31);
}

// C8 digests from the sets; set bytes (Fig. 10 footprint: live pairs and allocated capacity)
__global__ void k_plain_digest(PlainDev P) {
  const int lane = threadIdx.x & 31;
  const uint32_t nw = gridDim.x * (blockDim.x >> 5);
  for (uint32_t n = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); n < P.n_nodes; n += nw) {
    const SetDesc d = P.sets[n];
    const uint64_t hn = mix64p((uint64_t)n);
    unsigned long long s = 0;
    for (uint32_t i = lane; i < d.size; i += 32) s += mix64p(hn ^ P.heap[d.off + i]);
#pragma unroll
    for (int o = 16; o; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    if (lane == 0) {
      P.node_digest[n] = s;
      atomicAdd(P.app_digest, s);
      atomicAdd(&P.stats->alg_bytes, (unsigned long long)d.size * 8ull);
      atomicAdd(&P.stats->dense_bytes, (unsigned long long)d.cap * 8ull + sizeof(SetDesc));
    }
  }
}

// CELL -> node-major MAT store (readback and digests then use the MAT path's kernels): one
// warp per method, lanes over its cells; bit i of cell (r, c) -> word (r << logW) + c/64 of
// IN(node i).  Rows and columns are ordered as the node-major block's (locals, globals in gid
// order; sorted pool), so only the node changes.
__global__ void k_cell_to_mat(PlainDev P, Dev D, uint32_t M) {
  const int lane = threadIdx.x & 31;
  const uint32_t nw = gridDim.x * (blockDim.x >> 5);
  for (uint32_t m = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); m < M; m += nw) {
    const uint32_t rows = P.m_rows[m], cols = P.m_cols[m], wpc = P.m_wpc[m];
    const uint64_t ncell = (uint64_t)rows * cols;
    for (uint64_t q = lane; q < ncell; q += 32) {
      const uint32_t r = (uint32_t)(q / cols), c = (uint32_t)(q % cols);
      for (uint32_t w = 0; w < wpc; ++w) {
        uint64_t x = P.cells[P.m_coff[m] + q * wpc + w];
        while (x) {
          const int b = __ffsll((long long)x) - 1;
          x &= x - 1;
          const uint32_t node = P.mnodes[P.mnode_ptr[m] + w * 64 + b];
          const NodeRec R = D.nodes[node];
          atomicOr((unsigned long long*)(D.facts + R.off + ((uint64_t)r << R.logW) + (c >> 6)), 1ull << (c & 63));
          if (R.logW >= 1)                                  // wide block: row-occupancy bit (digest)
            atomicOr((unsigned long long*)(D.facts + R.off + ((R.B + 3u) & ~3u) + (r >> 6)), 1ull << (r & 63));
        }
      }
    }
  }
}

}  // namespace

cudaError_t launch_cell_to_mat(const PlainDev& P, const Dev& D, cudaStream_t s) {
  k_cell_to_mat<<<1184, 256, 0, s>>>(P, D, P.n_methods);
  return cudaGetLastError();
}

int plain_max_blocks(int device) {
  int sms = 0, occ = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device);
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_plain_fixpoint, 128, 0);
  return sms * (occ > 0 ? occ : 1);
}

cudaError_t launch_plain(const PlainDev& P, uint32_t blocks, cudaStream_t s) {
  k_plain_seed<<<1, 256, 0, s>>>(P);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return e;
  PlainDev p = P;
  void* args[] = {&p};
  return cudaLaunchCooperativeKernel((const void*)k_plain_fixpoint, dim3(blocks), dim3(128), args, 0, s);
}

cudaError_t launch_plain_digest(const PlainDev& P, cudaStream_t s) {
  k_plain_digest<<<1184, 256, 0, s>>>(P);
  return cudaGetLastError();
}

cudaError_t launch_plain_sizes(const PlainDev& P, uint32_t n0, uint32_t n1, uint64_t* out, cudaStream_t s) {
  k_plain_sizes<<<296, 256, 0, s>>>(P, n0, n1, out);
  return cudaGetLastError();
}

cudaError_t launch_plain_gather(const PlainDev& P, uint32_t n0, uint32_t n1, const uint64_t* ptr, uint64_t* pairs,
                                cudaStream_t s) {
  k_plain_gather<<<1184, 256, 0, s>>>(P, n0, n1, ptr, pairs);
  return cudaGetLastError();
}

}  // namespace gd
