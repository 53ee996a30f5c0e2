// layout.cu — (a1) device layout of a batch: the per-node and per-edge part of
// the load, as kernels over the uploaded descriptor arrays (Alg. 2 l.1-2 h_icfg / h_stmt ->
// d_icfg / d_stmt).  The host (loader.cu) validates and lays out the
// per-type / per-method / per-module tables only; everything that scales with nodes and edges —
// operand -> row resolution with V1 / V2 / V4, fact-block offsets (MAT), the
// (module, field) field-row tables, the cross-module projection tables π,
// edge records with V5 / V6, the GRP class sizes — runs here.
//
// Two phases, one host round trip between them (the totals size the field-row and projection
// tables):
//   k_dl_sizes   thread per node: CSR / kind / method / argument-range checks, target and kind of
//                every out-edge, padded block words, used (module, field) keys and (module, module)
//                pairs marked in dense per-app tables with their table sizes, work items per class;
//                then exclusive scans of the words, key sizes and pair sizes.
//   k_dl_nodes   thread per node: NodeRec (rows of every operand, fact offset, layout), argument
//                rows, global node-method / row_ptr / arg_ptr.
//   k_dl_frow    warp per used key: column -> global heap row of (column instance, field).
//   k_dl_xmap    warp per used module pair: colmap, rowmap, inverse rowmap (binary searches
//                in the sorted pools).
//   k_dl_edges   thread per node of out-degree <= 32: V5 / V6 of every out-edge, Edge records
//                with the destination layout and projection offset, inline chunk-0 records;
//                higher-degree nodes are listed for k_dl_edges_big (one warp per node).
//   k_dl_totals  the totals and the error word, stored into mapped pinned host memory.
// Errors never fault: every index read from the input is range-checked, and the first error
// (lowest app, then lowest node index) lands in err; the host then re-runs its own validator for
// the exact message (loader.cu).
#include "internal.cuh"

namespace gd {
namespace {

constexpr unsigned long long ERR_INVALID = 1, ERR_POOL = 2, ERR_LIMIT = 8;   // = -gdroid_status

__device__ __forceinline__ void dl_fail(const DLDev& L, uint32_t k, uint64_t idx, unsigned long long code) {
  atomicMin(L.err, ((unsigned long long)k << 44) | ((idx & ((1ull << 40) - 1)) << 4) | code);
}

// app of a global node id: the last app whose node_base <= n
__device__ __forceinline__ uint32_t app_of_node(const DLDev& L, uint32_t n) {
  uint32_t lo = 0, hi = L.n_apps - 1;
  while (lo < hi) {
    const uint32_t mid = (lo + hi + 1) >> 1;
    if (L.apps[mid].node_base <= n) lo = mid; else hi = mid - 1;
  }
  return lo;
}

// app of a dense-table entry j (keys: which = 0, pairs: 1): the last app whose base <= j
__device__ __forceinline__ uint32_t app_of_entry(const DLDev& L, uint64_t j, int which) {
  uint32_t lo = 0, hi = L.n_apps - 1;
  while (lo < hi) {
    const uint32_t mid = (lo + hi + 1) >> 1;
    const uint64_t b = which ? L.apps[mid].pair_base : L.apps[mid].key_base;
    if (b <= j) lo = mid; else hi = mid - 1;
  }
  return lo;
}

// index of key in the ascending a[0, n), -1 if absent
__device__ __forceinline__ int64_t dl_bsearch(const uint32_t* a, uint32_t n, uint32_t key) {
  uint32_t lo = 0, hi = n;
  while (lo < hi) {
    const uint32_t mid = (lo + hi) >> 1;
    if (a[mid] < key) lo = mid + 1; else hi = mid;
  }
  return (lo < n && a[lo] == key) ? (int64_t)lo : -1;
}

__global__ void __launch_bounds__(256) k_dl_sizes(DLDev L) {
  __shared__ uint32_t sc[NCLS];
  if (threadIdx.x < NCLS) sc[threadIdx.x] = 0;
  __syncthreads();
  const uint32_t stride = gridDim.x * blockDim.x;
  for (uint32_t n = blockIdx.x * blockDim.x + threadIdx.x; n < L.N; n += stride) {
    const uint32_t k = app_of_node(L, n);
    const DLApp& A = L.apps[k];
    const uint32_t i = n - A.node_base;
    const uint64_t r0 = L.rp[A.ptr_base + i], r1 = L.rp[A.ptr_base + i + 1];
    const uint64_t a0 = L.ap[A.ptr_base + i], a1 = L.ap[A.ptr_base + i + 1];
    const uint32_t kind = L.kind[n], lm = L.meth[n];
    L.words[n] = 0;
    // CSR monotone (with row_ptr[0] = 0 and row_ptr[N] = E checked on the host), kind, method
    if (r1 < r0 || r1 > A.n_edges || kind > GK_ASTORE || lm >= A.n_meths || a1 < a0 || a1 > A.n_args) {
      dl_fail(L, k, i, ERR_INVALID);
      continue;
    }
    const MethRec M = L.meths[A.meth_base + lm];
    const ModRec md = L.mods[M.module];
    bool bad = false;
    for (uint64_t e = r0; e < r1; ++e) {
      const uint32_t s = L.col[A.edge_base + e], ek = L.ekind[A.edge_base + e];
      if (s >= A.n_nodes || ek > GE_C2R) { dl_fail(L, k, (uint64_t)A.n_nodes + e, ERR_INVALID); bad = true; break; }
      if (ek == GE_CALL || ek == GE_RET) {                   // projection table of (src, dst) module
        const uint32_t tm = L.meth[A.node_base + s];
        if (tm >= A.n_meths) continue;                       // reported by the target's thread
        const uint32_t dm = L.meths[A.meth_base + tm].module;
        if (dm != M.module)
          L.psz[A.pair_base + (uint64_t)(M.module - A.mod_base) * A.n_mods + (dm - A.mod_base)] =
              md.n_cols + L.mods[dm].n_glob + md.n_glob;     // colmap, rowmap, inverse rowmap
      }
    }
    if (bad) continue;
    const uint64_t deg = r1 - r0, rows = (uint64_t)M.n_locals + md.n_glob, B = rows << md.logW;
    if (B >= (1ull << 32) || M.n_locals > 0xffff || (md.logW >= 1 && rows > 1024) || deg > 32768) {
      dl_fail(L, k, i, ERR_LIMIT);
      continue;
    }
    uint64_t w = (B + 3) & ~3ull;                             // 32-byte aligned blocks
    if (md.logW >= 1) w += (occ_words((uint32_t)rows) + 3) & ~3ull;   // wide: row-occupancy words
    L.words[n] = (uint32_t)w;
    if (kind >= GK_FLOAD) {                                   // FLOAD FSTORE ALOAD ASTORE
      const int32_t f = (kind == GK_ALOAD || kind == GK_ASTORE) ? (int32_t)GDROID_F_ARR : L.ops[4ull * n + 2];
      if (f >= 0 && (uint32_t)f < A.n_fields)
        L.ksz[A.key_base + (uint64_t)(M.module - A.mod_base) * A.n_fields + (uint32_t)f] = md.n_cols;
    }
    const uint32_t c = kind_cls(kind);
    atomicAdd(&sc[c], n_chunks_of((uint32_t)deg, c, md.logW));
  }
  __syncthreads();
  if (threadIdx.x < NCLS && sc[threadIdx.x]) atomicAdd(&L.cls[threadIdx.x], sc[threadIdx.x]);
}

__global__ void __launch_bounds__(256) k_dl_nodes(DLDev L) {
  const uint32_t stride = gridDim.x * blockDim.x;
  for (uint32_t n = blockIdx.x * blockDim.x + threadIdx.x; n < L.N; n += stride) {
    const uint32_t k = app_of_node(L, n);
    const DLApp& A = L.apps[k];
    const uint32_t i = n - A.node_base;
    const uint32_t kind = L.kind[n], lm = L.meth[n];
    if (n == 0) { L.rowptr[0] = 0; L.argptr[0] = 0; }
    if (kind > GK_ASTORE || lm >= A.n_meths) continue;      // reported by k_dl_sizes
    const uint64_t r0 = L.rp[A.ptr_base + i], r1 = L.rp[A.ptr_base + i + 1];
    const uint64_t a0 = L.ap[A.ptr_base + i], a1 = L.ap[A.ptr_base + i + 1];
    if (a1 < a0 || a1 > A.n_args || r1 < r0 || r1 > A.n_edges) continue;
    const MethRec M = L.meths[A.meth_base + lm];
    const ModRec md = L.mods[M.module];
    const int32_t* op = L.ops + 4ull * n;
    const uint32_t Lr = M.n_locals;
    NodeRec R{};
    R.kind = (uint8_t)kind; R.cls = (uint8_t)kind_cls(kind); R.app = (uint16_t)k;
    R.r0 = R.r1 = R.r2 = R.r3 = -1;
    unsigned long long err = 0;
    auto local = [&](int32_t gid, int32_t& out) {             // V4: operand is a local of the method
      const int64_t v = (int64_t)gid - (int64_t)M.local_base;
      if (v < 0 || v >= (int64_t)Lr) { if (!err) err = ERR_POOL; return; }
      out = (int32_t)v;
    };
    auto static_row = [&](int32_t gid, int32_t& out) {        // V2: static visible in the module
      if (gid < (int64_t)A.stat_lo || gid >= (int64_t)A.stat_hi) { if (!err) err = ERR_INVALID; return; }
      const int64_t pos = dl_bsearch(L.grow_gid + md.grow_off, md.n_stat, (uint32_t)gid);
      if (pos < 0) { if (!err) err = ERR_POOL; return; }
      out = (int32_t)(Lr + pos);
    };
    switch (kind) {
      case GK_PRIM: local(op[0], R.r0); break;
      case GK_CONST: case GK_NEW: {
        local(op[0], R.r0);
        if (err) break;
        if (op[3] < 0 || (uint32_t)op[3] >= A.n_inst || (kind == GK_NEW && op[3] == 0)) { err = ERR_INVALID; break; }
        const int64_t c = dl_bsearch(L.col_gid + md.col_off, md.n_cols, (uint32_t)op[3]);   // V1
        if (c < 0) { err = ERR_POOL; break; }
        R.r3 = (int32_t)c;
        break;
      }
      case GK_COPY: local(op[0], R.r0); local(op[1], R.r1); break;
      case GK_FLOAD: case GK_FSTORE: case GK_ALOAD: case GK_ASTORE: {
        local(op[0], R.r0); local(op[1], R.r1);
        if (err) break;
        int32_t f = (int32_t)GDROID_F_ARR;
        if (kind == GK_FLOAD || kind == GK_FSTORE) {
          if (op[2] < 0 || (uint32_t)op[2] >= A.n_fields) { err = ERR_INVALID; break; }
          f = op[2];
        }
        R.r2 = f;
        if ((uint32_t)f < A.n_fields)                          // field-row table of (module, f)
          R.r3 = (int32_t)L.koff[A.key_base + (uint64_t)(M.module - A.mod_base) * A.n_fields + (uint32_t)f];
        break;
      }
      case GK_SLOAD: local(op[0], R.r0); if (!err) static_row(op[1], R.r1); break;
      case GK_SSTORE: local(op[1], R.r1); if (!err) static_row(op[0], R.r0); break;
      case GK_RETV: local(op[1], R.r1); R.r0 = (int32_t)(Lr - 1); break;   // RET_m
      case GK_CALL: if (op[0] >= 0) local(op[0], R.r0); break;
      case GK_RETSITE: {
        const int32_t c = op[3];
        if (c < 0 || (uint32_t)c >= A.n_nodes || L.kind[A.node_base + c] != GK_CALL ||
            L.meth[A.node_base + c] != lm || L.ops[4ull * (A.node_base + c)] != op[0]) { err = ERR_INVALID; break; }
        if (op[0] >= 0) local(op[0], R.r0);
        break;
      }
      default: break;
    }
    if (!err && kind != GK_CALL && a1 != a0) err = ERR_INVALID;   // arguments on a non-CALL node
    if (!err) {
      for (uint64_t q = a0; q < a1; ++q) {
        int32_t row = -1;
        const int32_t g = L.cargs[A.arg_base + q];
        if (g >= 0) local(g, row);
        L.args[A.arg_base + q] = row;
        if (kind == GK_CALL && a1 - a0 <= 3) (&R.r1)[q - a0] = row;   // inline argument rows
      }
    }
    if (err) { dl_fail(L, k, i, err); continue; }
    if (kind == GK_ENTRY) R.r1 = (int32_t)M.n_params;
    R.off = L.foff[n];
    R.B = (Lr + md.n_glob) << md.logW;
    R.L = Lr; R.n_stat = md.n_stat;
    R.e0 = A.edge_base + (uint32_t)r0; R.e1 = A.edge_base + (uint32_t)r1;
    R.col_off = md.col_off; R.grow_off = md.grow_off; R.n_cols = (uint16_t)md.n_cols;
    R.logW = (uint8_t)md.logW; R.local_base = M.local_base;
    L.nodes[n] = R;
    L.nodemeth[n] = A.meth_base + lm;
    L.rowptr[n + 1] = A.edge_base + (uint32_t)r1;
    L.argptr[n + 1] = A.arg_base + (uint32_t)a1;
  }
}

// field-row table of one used (module, field) key: column c -> global row of (Q[c], f) or -1
// One warp per 32 consecutive key entries; every used key's table is filled by the whole warp
// (lanes over the columns).
__global__ void __launch_bounds__(256) k_dl_frow(DLDev L) {
  const uint32_t lane = threadIdx.x & 31;
  const uint64_t nwarp = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  for (uint64_t j0 = (((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5) * 32; j0 < L.K; j0 += nwarp * 32) {
    const uint64_t jl = j0 + lane;
    unsigned used = __ballot_sync(0xffffffffu, jl < L.K && L.ksz[jl] != 0);
    while (used) {
      const uint64_t j = j0 + (__ffs(used) - 1);
      used &= used - 1;
      const DLApp& A = L.apps[app_of_entry(L, j, 0)];
      const uint64_t loc = j - A.key_base;
      const uint32_t d = (uint32_t)(loc / A.n_fields), f = (uint32_t)(loc % A.n_fields);
      const ModRec md = L.mods[A.mod_base + d];
      int32_t* out = L.frow + L.koff[j];
      for (uint32_t c = lane; c < md.n_cols; c += 32) {
        const int32_t ty = L.col_type[md.col_off + c];
        int32_t row = -1;
        if (c != 0 && ty >= 0)
          for (uint32_t q = L.tf_ptr[ty]; q < L.tf_ptr[ty + 1]; ++q)
            if (L.tf[q] == f) row = (int32_t)(L.col_hbase[md.col_off + c] + (q - L.tf_ptr[ty]));
        out[c] = row;
      }
    }
  }
}

// projection table π of one (source module, target module) pair: a column
// is kept iff its instance is in Q_dst, a global row iff its slot is in P_src.  colmap[|Q_src|]
// (src column -> dst column), rowmap[n_glob(dst)] (dst global row -> src global row), inverse
// rowmap[n_glob(src)]; -1 = dropped.  One warp per 32 consecutive pair entries; a used pair's
// table is filled by the whole warp: -1 everywhere, then lanes over the target's columns and
// statics, each found in the source's ascending pool by binary search.
__global__ void __launch_bounds__(256) k_dl_xmap(DLDev L) {
  const uint32_t lane = threadIdx.x & 31;
  const uint64_t nwarp = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  for (uint64_t j0 = (((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5) * 32; j0 < L.P; j0 += nwarp * 32) {
    const uint64_t jl = j0 + lane;
    unsigned used = __ballot_sync(0xffffffffu, jl < L.P && L.psz[jl] != 0);
    while (used) {
      const uint64_t j = j0 + (__ffs(used) - 1);
      used &= used - 1;
      const uint32_t sz = L.psz[j];
      const DLApp& A = L.apps[app_of_entry(L, j, 1)];
      const uint64_t loc = j - A.pair_base;
      const ModRec ms = L.mods[A.mod_base + (uint32_t)(loc / A.n_mods)];
      const ModRec mt = L.mods[A.mod_base + (uint32_t)(loc % A.n_mods)];
      int32_t* cmap = L.xmap + L.poff[j];
      int32_t* rmap = cmap + ms.n_cols;
      int32_t* rinv = rmap + mt.n_glob;
      for (uint32_t q = lane; q < sz; q += 32) cmap[q] = -1;
      __syncwarp();                                            // the -1 fill before the entries
      const uint32_t* Ps = L.col_gid + ms.col_off;
      for (uint32_t b = lane; b < mt.n_cols; b += 32) {       // instances of Q_dst found in Q_src
        const int64_t a = dl_bsearch(Ps, ms.n_cols, L.col_gid[mt.col_off + b]);
        if (a < 0) continue;
        cmap[a] = (int32_t)b;
        const int32_t ty = L.col_type[mt.col_off + b];       // heap rows of a shared instance
        if (b != 0 && ty >= 0) {
          const uint32_t nf = L.tf_ptr[ty + 1] - L.tf_ptr[ty];
          const uint32_t gt = L.col_hbase[mt.col_off + b], gs = L.col_hbase[ms.col_off + (uint32_t)a];
          for (uint32_t q = 0; q < nf; ++q) { rmap[gt + q] = (int32_t)(gs + q); rinv[gs + q] = (int32_t)(gt + q); }
        }
      }
      const uint32_t* Ss = L.grow_gid + ms.grow_off;        // static rows: ascending slot gids
      for (uint32_t b = lane; b < mt.n_stat; b += 32) {
        const int64_t a = dl_bsearch(Ss, ms.n_stat, L.grow_gid[mt.grow_off + b]);
        if (a >= 0) { rmap[b] = (int32_t)a; rinv[a] = (int32_t)b; }
      }
      __syncwarp();
    }
  }
}

// V5 / V6 of out-edge el of node n (app-local i), and its Edge record (destination layout copied
// in; CALL aux = the callee's n_params, RET aux = lhs(c) row at the return site).  Returns 0 or the
// error code.
struct EdgeCtx {
  uint32_t n, i, kind, lm, sm, my_entry;
  uint64_t a0, a1;
};
__device__ __forceinline__ unsigned long long dl_edge(const DLDev& L, const DLApp& A, const EdgeCtx& c, uint64_t el,
                                                      uint32_t& ek_out, Edge& E2) {
  const uint64_t e = A.edge_base + el;
  const uint32_t sl = L.col[e], ek = L.ekind[e];
  ek_out = ek;
  if (sl >= A.n_nodes || ek > GE_C2R) return ERR_INVALID;
  const uint32_t s = A.node_base + sl, skind = L.kind[s], tm = L.meth[s];
  if (tm >= A.n_meths) return ERR_INVALID;
  bool ok = true;
  switch (ek) {
    case GE_INTRA: ok = c.kind != GK_CALL && c.kind != GK_EXIT && tm == c.lm; break;
    case GE_C2R: ok = c.kind == GK_CALL && skind == GK_RETSITE && L.ops[4ull * s + 3] == (int32_t)c.i; break;
    case GE_CALL:                                              // V5 + V6 (arity)
      ok = c.kind == GK_CALL && skind == GK_ENTRY && L.mentry[A.meth_base + tm] == sl &&
           c.a1 - c.a0 == L.meths[A.meth_base + tm].n_params;
      break;
    case GE_RET: {                                             // to a site that calls this method
      ok = c.kind == GK_EXIT && skind == GK_RETSITE;
      const int32_t cs = ok ? L.ops[4ull * s + 3] : -1;
      if (ok && (cs < 0 || (uint32_t)cs >= A.n_nodes)) ok = false;
      if (ok) {
        const uint64_t c0 = L.rp[A.ptr_base + cs], c1 = L.rp[A.ptr_base + cs + 1];
        bool found = false;
        if (c1 >= c0 && c1 <= A.n_edges)
          for (uint64_t e2 = c0; e2 < c1 && !found; ++e2)
            found = L.ekind[A.edge_base + e2] == GE_CALL && L.col[A.edge_base + e2] == c.my_entry;
        ok = found;
      }
      break;
    }
  }
  if (!ok) return ERR_INVALID;
  uint32_t xoff = NO_XMAP;
  if (ek == GE_CALL || ek == GE_RET) {
    const uint32_t dm = L.meths[A.meth_base + tm].module;
    if (dm != c.sm) xoff = (uint32_t)L.poff[A.pair_base + (uint64_t)(c.sm - A.mod_base) * A.n_mods + (dm - A.mod_base)];
  }
  const NodeRec RS = L.nodes[s];
  const uint32_t nch = n_chunks_of(RS.e1 - RS.e0, RS.cls, RS.logW);
  E2.dst = s;
  E2.info = ek | ((uint32_t)RS.cls << 2) | ((nch - 1) << 5) | (RS.logW >= 1 ? INFO_WIDE : 0u);
  E2.off = RS.off; E2.B = RS.B; E2.L = (uint16_t)RS.L; E2.logW = RS.logW; E2.pad = 0;
  E2.aux = ek == GE_CALL ? RS.r1 : (ek == GE_RET ? RS.r0 : -1);
  E2.xoff = xoff;
  L.edges[e] = E2;
  return 0;
}

// Node n's edge context; false if k_dl_sizes already rejected the node.
__device__ __forceinline__ bool dl_edge_ctx(const DLDev& L, uint32_t n, uint32_t& k, EdgeCtx& c, uint64_t& r0, uint64_t& r1) {
  k = app_of_node(L, n);
  const DLApp& A = L.apps[k];
  c.n = n; c.i = n - A.node_base;
  c.kind = L.kind[n]; c.lm = L.meth[n];
  if (c.kind > GK_ASTORE || c.lm >= A.n_meths) return false;
  r0 = L.rp[A.ptr_base + c.i]; r1 = L.rp[A.ptr_base + c.i + 1];
  c.a0 = L.ap[A.ptr_base + c.i]; c.a1 = L.ap[A.ptr_base + c.i + 1];
  if (r1 < r0 || r1 > A.n_edges || c.a1 < c.a0 || c.a1 > A.n_args || r1 - r0 > 32768) return false;
  c.sm = L.meths[A.meth_base + c.lm].module;
  c.my_entry = L.mentry[A.meth_base + c.lm];
  return true;
}

// Inline chunk-0 records: chunk 0 goes inline when it holds only INTRA / C2R edges of a narrow
// block of <= INL_MAX_B words (as k_edges of kernels.cu).
constexpr uint32_t DL_WARP_DEG = 32;     // nodes with more out-edges: one warp each (k_dl_edges_big)

// V5 / V6 and Edge records, thread per node of out-degree <= DL_WARP_DEG; the others are listed in
// big[] for k_dl_edges_big.
__global__ void __launch_bounds__(256) k_dl_edges(DLDev L, uint32_t* big, uint32_t* n_big) {
  const uint32_t stride = gridDim.x * blockDim.x;
  for (uint32_t n = blockIdx.x * blockDim.x + threadIdx.x; n < L.N; n += stride) {
    uint32_t k;
    EdgeCtx c;
    uint64_t r0, r1;
    if (!dl_edge_ctx(L, n, k, c, r0, r1)) continue;
    const uint32_t deg = (uint32_t)(r1 - r0);
    if (deg > DL_WARP_DEG) { big[atomicAdd(n_big, 1u)] = n; continue; }
    const DLApp& A = L.apps[k];
    const NodeRec R = L.nodes[n];
    const uint32_t n0 = min(deg, chunk_edges(deg, R.cls, R.logW));
    bool inl_ok = deg > 0 && n0 <= 4 && R.logW == 0 && R.B <= INL_MAX_B;
    InlEdge rec[4];
    uint32_t n_c2r = 0;
    unsigned long long err = 0;
    uint64_t err_e = 0;
    for (uint64_t el = r0; el < r1; ++el) {
      uint32_t ek;
      Edge E2;
      err = dl_edge(L, A, c, el, ek, E2);
      if (err) { err_e = el; break; }
      n_c2r += ek == GE_C2R;
      const uint32_t jj = (uint32_t)(el - r0);
      if (jj < 4) rec[jj] = InlEdge{E2.dst, E2.info, E2.off};
      if (jj < n0) inl_ok = inl_ok && (ek == GE_INTRA || ek == GE_C2R);
    }
    if (!err && c.kind == GK_CALL && n_c2r != 1) { err = ERR_INVALID; err_e = ~0ull; }
    if (err) {
      dl_fail(L, k, err_e == ~0ull ? c.i : (uint64_t)A.n_nodes + err_e, err);
      continue;
    }
    for (uint32_t j = 0; j < 4; ++j) L.inl[4ull * n + j] = (inl_ok && j < n0) ? rec[j] : InlEdge{0u, 0u, 0ull};
    L.nodes[n].n_inl = inl_ok ? (uint8_t)n0 : (uint8_t)0;   // (other threads read other fields only)
  }
}

// The same for the listed high-degree nodes (method exits with many return sites, virtual calls
// with many targets), one warp per node, lanes over the edges.
__global__ void __launch_bounds__(256) k_dl_edges_big(DLDev L, const uint32_t* big, const uint32_t* n_big) {
  const uint32_t lane = threadIdx.x & 31, nb = *n_big;
  const uint32_t stride = (gridDim.x * blockDim.x) >> 5;
  for (uint32_t w = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; w < nb; w += stride) {
    const uint32_t n = big[w];
    uint32_t k;
    EdgeCtx c;
    uint64_t r0, r1;
    dl_edge_ctx(L, n, k, c, r0, r1);                          // listed: the checks passed
    const DLApp& A = L.apps[k];
    const NodeRec R = L.nodes[n];
    const uint32_t deg = (uint32_t)(r1 - r0), n0 = min(deg, chunk_edges(deg, R.cls, R.logW));
    bool inl_ok = n0 <= 4 && R.logW == 0 && R.B <= INL_MAX_B;
    uint32_t n_c2r = 0;
    unsigned long long err_w = ~0ull;                          // (edge index << 4 | code), lowest wins
    InlEdge rec{0u, 0u, 0ull};
    bool rec_ok = true;
    for (uint64_t el = r0 + lane; el < r1; el += 32) {
      uint32_t ek;
      Edge E2;
      const unsigned long long err = dl_edge(L, A, c, el, ek, E2);
      if (err) { err_w = min(err_w, ((el - r0) << 4) | err); continue; }
      n_c2r += ek == GE_C2R;
      const uint32_t jj = (uint32_t)(el - r0);
      if (jj < 4) rec = InlEdge{E2.dst, E2.info, E2.off};
      if (jj < n0) rec_ok = ek == GE_INTRA || ek == GE_C2R;
    }
    for (int o = 16; o; o >>= 1) {
      err_w = min(err_w, (unsigned long long)__shfl_xor_sync(0xffffffffu, err_w, o));
      n_c2r += __shfl_xor_sync(0xffffffffu, n_c2r, o);
    }
    inl_ok = inl_ok && __all_sync(0xffffffffu, rec_ok);
    if (err_w == ~0ull && c.kind == GK_CALL && n_c2r != 1) err_w = (1ull << 44) | ERR_INVALID;
    if (err_w != ~0ull) {
      if (lane == 0) {
        const uint64_t el = err_w >> 4;
        dl_fail(L, k, el >= (1ull << 40) ? c.i : (uint64_t)A.n_nodes + r0 + el, err_w & 15);
      }
      continue;
    }
    if (lane < 4) L.inl[4ull * n + lane] = (inl_ok && lane < n0) ? rec : InlEdge{0u, 0u, 0ull};
    if (lane == 0) L.nodes[n].n_inl = inl_ok ? (uint8_t)n0 : (uint8_t)0;
  }
}

// totals of the layout for the host, stored into mapped pinned memory: fact words, field-row and
// projection table sizes, the error word, class counts (two per word)
__global__ void k_dl_totals(DLDev L, uint64_t* out) {
  if (threadIdx.x != 0) return;
  out[0] = L.foff[L.N];
  out[1] = L.koff[L.K];
  out[2] = L.poff[L.P];
  out[3] = *L.err;
  for (int c = 0; c < NCLS; c += 2)
    out[4 + c / 2] = (uint64_t)L.cls[c] | (c + 1 < NCLS ? (uint64_t)L.cls[c + 1] << 32 : 0ull);
  __threadfence_system();
}

uint32_t grid_for(uint64_t n) {
  uint64_t b = (n + 255) / 256;
  return (uint32_t)(b == 0 ? 1 : (b > 148 * 8 ? 148 * 8 : b));
}

}  // namespace

cudaError_t launch_dl_sizes(const DLDev& L, uint64_t* scan_tmp, cudaStream_t s) {
  k_dl_sizes<<<grid_for(L.N), 256, 0, s>>>(L);
  cudaError_t e = launch_scan_counts(L.words, L.N, L.foff, scan_tmp, s);
  if (e == cudaSuccess) e = launch_scan_counts(L.ksz, (uint32_t)L.K, L.koff, scan_tmp, s);
  if (e == cudaSuccess) e = launch_scan_counts(L.psz, (uint32_t)L.P, L.poff, scan_tmp, s);
  return e != cudaSuccess ? e : cudaGetLastError();
}

cudaError_t launch_dl_totals(const DLDev& L, uint64_t* host_mapped, cudaStream_t s) {
  k_dl_totals<<<1, 32, 0, s>>>(L, host_mapped);
  return cudaGetLastError();
}

cudaError_t launch_dl_records(const DLDev& L, cudaStream_t s) {
  k_dl_nodes<<<grid_for(L.N), 256, 0, s>>>(L);
  if (L.K) k_dl_frow<<<grid_for((L.K + 31) / 32 * 32), 256, 0, s>>>(L);
  if (L.P) k_dl_xmap<<<grid_for((L.P + 31) / 32 * 32), 256, 0, s>>>(L);
  // the high-degree list reuses the phase-1 words[] (scan input, dead by now); its counter sits
  // in cls[8] (zeroed with the class counts)
  k_dl_edges<<<grid_for(L.N), 256, 0, s>>>(L, L.words, L.cls + 8);
  k_dl_edges_big<<<148 * 8, 256, 0, s>>>(L, L.words, L.cls + 8);
  return cudaGetLastError();
}

}  // namespace gd
