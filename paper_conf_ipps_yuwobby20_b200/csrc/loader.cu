// loader.cu — host side of libgdroid.so: the C ABI of include/gdroid.h.
//
// (a1) validates each app's ICFG (V1-V6 of DESIGN.md §3), resolves every operand to a row of
// its node's fact block, lays out the fact store (node-major MAT blocks),
// builds the cross-module projection tables and uploads everything with one pinned staging
// buffer (the paper's dual-buffered copy, Alg. 2 l.2, is recast as the corpus driver's
// double-buffered per-batch H2D).  (a2)-(a7) are enqueued by gdroid_build_idfg.
#include <algorithm>
#include <chrono>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <map>
#include <string>
#include <vector>

#include "internal.cuh"

using namespace gd;

namespace {

thread_local std::string g_err;

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

// Host images of every device table of a batch.
struct HostImage {
  std::vector<NodeRec> nodes;
  std::vector<MethRec> meths;
  std::vector<ModRec> mods;
  std::vector<uint32_t> row_ptr{0};
  std::vector<Edge> edges;
  std::vector<uint32_t> arg_ptr{0};
  std::vector<int32_t> args;
  std::vector<uint32_t> col_gid, col_hbase;
  std::vector<int32_t> col_type;
  std::vector<uint32_t> grow_gid;
  std::vector<int32_t> grow_col, grow_field;
  std::vector<uint32_t> tf_ptr{0}, tf;
  std::vector<int32_t> xmap;                   // projection tables: colmap then rowmap
  std::vector<int32_t> frow;                   // per (module, field): column -> global heap row | -1
  std::vector<uint32_t> app_node_base;
  std::vector<uint32_t> entries;
  std::vector<uint32_t> node_method;
  uint64_t fact_words = 0;
  uint32_t cls_count[NCLS] = {0, 0, 0, 0, 0};
};

// Per-module host-side lookup info of the app being loaded.
struct ModInfo {
  const uint32_t* insts; uint64_t n_insts;
  const uint32_t* stats; uint64_t n_stats;
  uint32_t gmod;   // global module index
};

gdroid_status add_app(HostImage& H, const gdroid_icfg_desc* d, uint32_t k) {
  if (!d) return set_err(GDROID_E_INVALID, "app %u: NULL descriptor", k);
  if (d->abi_version != GDROID_ABI_VERSION)
    return set_err(GDROID_E_INVALID, "app %u: abi_version %u != %u", k, d->abi_version, GDROID_ABI_VERSION);
  const uint64_t N = d->n_nodes, E = d->n_edges, M = d->n_methods, Dm = d->n_modules;
  const uint64_t I = d->n_instances, G = d->n_statics, T = d->n_types;
  if (N == 0 || M == 0 || Dm == 0 || I == 0) return set_err(GDROID_E_INVALID, "app %u: empty ICFG", k);
  if ((uint64_t)H.nodes.size() + N >= (1ull << 32) || (uint64_t)H.edges.size() + E >= (1ull << 32))
    return set_err(GDROID_E_LIMIT, "app %u: batch exceeds 2^32 nodes or edges", k);
  const uint32_t nb = (uint32_t)H.nodes.size(), mb = (uint32_t)H.meths.size();
  const uint32_t db = (uint32_t)H.mods.size(), tb = (uint32_t)(H.tf_ptr.size() - 1);
  // ---- CSR (structure)
  if (d->row_ptr[0] != 0) return set_err(GDROID_E_INVALID, "app %u: row_ptr[0] != 0", k);
  for (uint64_t n = 0; n < N; ++n)
    if (d->row_ptr[n + 1] < d->row_ptr[n]) return set_err(GDROID_E_INVALID, "app %u: row_ptr not monotone at node %llu", k, (unsigned long long)n);
  if (d->row_ptr[N] != E) return set_err(GDROID_E_INVALID, "app %u: row_ptr[n_nodes] != n_edges", k);
  for (uint64_t e = 0; e < E; ++e) {
    if (d->col[e] >= N) return set_err(GDROID_E_INVALID, "app %u: edge %llu target out of range", k, (unsigned long long)e);
    if (d->edge_kind[e] > GE_C2R) return set_err(GDROID_E_INVALID, "app %u: edge %llu bad kind", k, (unsigned long long)e);
  }
  for (uint64_t n = 0; n < N; ++n) {
    if (d->node_kind[n] > GK_ASTORE) return set_err(GDROID_E_INVALID, "app %u: node %llu bad kind", k, (unsigned long long)n);
    if (d->node_method[n] >= M) return set_err(GDROID_E_INVALID, "app %u: node %llu method out of range", k, (unsigned long long)n);
  }
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
  std::vector<uint64_t> heap_base(I + 1, 0);
  for (uint64_t o = 0; o < I; ++o) {
    const int32_t t = d->inst_type[o];
    if (t < -1 || t >= (int64_t)T) return set_err(GDROID_E_INVALID, "app %u: instance %llu type out of range", k, (unsigned long long)o);
    heap_base[o + 1] = heap_base[o] + (t < 0 ? 0 : d->type_field_ptr[t + 1] - d->type_field_ptr[t]);
  }
  // ---- methods / slot numbering
  std::vector<uint64_t> local_base(M + 1, 0);
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
  // ---- modules: pools, rows, columns
  std::vector<ModInfo> mi(Dm);
  for (uint64_t dd = 0; dd < Dm; ++dd) {
    const uint64_t a = d->module_inst_ptr[dd], b = d->module_inst_ptr[dd + 1];
    const uint64_t sa = d->module_static_ptr[dd], sb = d->module_static_ptr[dd + 1];
    if (b < a || sb < sa) return set_err(GDROID_E_INVALID, "app %u: module %llu pool CSR not monotone", k, (unsigned long long)dd);
    if (b == a || d->module_insts[a] != 0) return set_err(GDROID_E_POOL, "app %u: module %llu pool lacks NULL", k, (unsigned long long)dd);
    for (uint64_t q = a; q < b; ++q) {
      if (d->module_insts[q] >= I) return set_err(GDROID_E_INVALID, "app %u: module %llu instance out of range", k, (unsigned long long)dd);
      if (q > a && d->module_insts[q] <= d->module_insts[q - 1]) return set_err(GDROID_E_INVALID, "app %u: module %llu pool not strictly ascending", k, (unsigned long long)dd);
    }
    for (uint64_t q = sa; q < sb; ++q) {
      if (d->module_statics[q] >= G) return set_err(GDROID_E_INVALID, "app %u: module %llu static out of range", k, (unsigned long long)dd);
      if (q > sa && d->module_statics[q] <= d->module_statics[q - 1]) return set_err(GDROID_E_INVALID, "app %u: module %llu statics not strictly ascending", k, (unsigned long long)dd);
    }
    const uint64_t ncol = b - a;
    if (ncol > 64ull * MAXW) return set_err(GDROID_E_LIMIT, "app %u: module %llu pool has %llu > %d instances", k, (unsigned long long)dd, (unsigned long long)ncol, 64 * MAXW);
    uint32_t W = 1, logW = 0;
    while (64ull * W < ncol) { W <<= 1; ++logW; }
    ModRec md{};
    md.n_cols = (uint32_t)ncol; md.W = W; md.logW = logW;
    md.n_stat = (uint32_t)(sb - sa);
    md.col_off = (uint32_t)H.col_gid.size();
    md.grow_off = (uint32_t)H.grow_gid.size();
    for (uint64_t q = sa; q < sb; ++q) {                       // static rows
      H.grow_gid.push_back((uint32_t)(Lt + d->module_statics[q]));
      H.grow_col.push_back(-1); H.grow_field.push_back(-1);
    }
    uint32_t hrow = md.n_stat;
    for (uint64_t c = 0; c < ncol; ++c) {                      // columns + heap rows
      const uint32_t o = d->module_insts[a + c];
      const int32_t t = d->inst_type[o];
      H.col_gid.push_back(o);
      H.col_type.push_back(t < 0 ? -1 : (int32_t)(tb + t));
      H.col_hbase.push_back(hrow);
      if (t >= 0) {
        for (uint64_t q = d->type_field_ptr[t]; q < d->type_field_ptr[t + 1]; ++q) {
          H.grow_gid.push_back((uint32_t)(Lt + G + heap_base[o] + (q - d->type_field_ptr[t])));
          H.grow_col.push_back((int32_t)c);
          H.grow_field.push_back((int32_t)d->type_fields[q]);
          ++hrow;
        }
      }
    }
    md.n_glob = hrow;
    H.mods.push_back(md);
    mi[dd] = ModInfo{d->module_insts + a, ncol, d->module_statics + sa, sb - sa, db + (uint32_t)dd};
  }
  for (uint64_t m = 0; m < M; ++m)
    H.meths.push_back(MethRec{d->method_n_locals[m], d->method_n_params[m], db + d->method_module[m], (uint32_t)local_base[m]});
  // ---- nodes: operands -> rows (V1, V2, V4), fact offsets
  H.app_node_base.push_back(nb);
  std::map<std::pair<uint32_t, uint32_t>, uint32_t> frow_map;
  auto local_idx = [&](int64_t gid, uint64_t m) -> int64_t {
    if (gid < (int64_t)local_base[m] || gid >= (int64_t)local_base[m + 1]) return -1;
    return gid - (int64_t)local_base[m];
  };
  for (uint64_t n = 0; n < N; ++n) {
    const uint8_t kind = d->node_kind[n];
    const uint64_t m = d->node_method[n];
    const uint64_t dd = d->method_module[m];
    const ModInfo& P = mi[dd];
    const ModRec& md = H.mods[db + dd];
    const uint32_t L = d->method_n_locals[m];
    const int32_t* op = d->node_ops + 4 * n;
    NodeRec R{};
    R.kind = kind; R.cls = (uint8_t)cls_of(kind); R.app = (uint16_t)k;
    H.node_method.push_back(mb + (uint32_t)m);
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
        if (kind == GK_FLOAD || kind == GK_ALOAD) {          // heap row of (o1, f) per column
          auto key = std::make_pair((uint32_t)dd, (uint32_t)R.r2);
          auto it = frow_map.find(key);
          if (it == frow_map.end()) {
            const uint32_t off = (uint32_t)H.frow.size();
            for (uint32_t c = 0; c < md.n_cols; ++c) {
              const int32_t ty = H.col_type[md.col_off + c];
              int32_t row = -1;
              if (c != 0 && ty >= 0)
                for (uint32_t q = H.tf_ptr[ty]; q < H.tf_ptr[ty + 1]; ++q)
                  if (H.tf[q] == (uint32_t)R.r2) row = (int32_t)(H.col_hbase[md.col_off + c] + (q - H.tf_ptr[ty]));
              H.frow.push_back(row);
            }
            it = frow_map.emplace(key, off).first;
          }
          R.r3 = (int32_t)it->second;
        }
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
    if (a1 < a0) return set_err(GDROID_E_INVALID, "app %u: call_arg_ptr not monotone at %llu", k, (unsigned long long)n);
    if (kind != GK_CALL && a1 != a0) return set_err(GDROID_E_INVALID, "app %u: node %llu: arguments on a non-CALL node", k, (unsigned long long)n);
    for (uint64_t q = a0; q < a1; ++q) {
      int32_t row = -1;
      if (d->call_args[q] >= 0 && !need_local(d->call_args[q], row, "argument")) return GDROID_E_POOL;
      H.args.push_back(row);
      if (kind == GK_CALL && a1 - a0 <= 3) (&R.r1)[q - a0] = row;   // inline argument rows
    }
    H.arg_ptr.push_back((uint32_t)H.args.size());
    if (kind == GK_ENTRY) R.r1 = (int32_t)d->method_n_params[m];
    R.off = H.fact_words;
    const uint64_t words = (uint64_t)(L + md.n_glob) << md.logW;
    if (words >= (1ull << 32)) return set_err(GDROID_E_LIMIT, "app %u: node %llu: fact block too large", k, (unsigned long long)n);
    R.B = (uint32_t)words; R.L = L; R.n_stat = md.n_stat;
    R.e0 = (uint32_t)(H.edges.size() + d->row_ptr[n]); R.e1 = (uint32_t)(H.edges.size() + d->row_ptr[n + 1]);
    R.col_off = md.col_off; R.grow_off = md.grow_off; R.n_cols = (uint16_t)md.n_cols;
    R.logW = (uint8_t)md.logW; R.module = db + (uint32_t)dd;
    H.fact_words += (words + 3) & ~3ull;                        // 32-byte aligned blocks
    H.nodes.push_back(R);
  }
  // ---- edges (V5, V6) + projection tables
  std::map<std::pair<uint32_t, uint32_t>, uint32_t> xmap;   // (src module, dst module) -> xoff
  for (uint64_t n = 0; n < N; ++n) {
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
          auto key = std::make_pair(db + sm, db + dm);
          auto it = xmap.find(key);
          if (it != xmap.end()) xoff = it->second;
          else {
            xoff = (uint32_t)H.xmap.size();
            xmap[key] = xoff;
            const ModRec &ms = H.mods[db + sm], &mt = H.mods[db + dm];
            for (uint32_t c = 0; c < ms.n_cols; ++c) {      // columns: instance kept iff in Q_dst
              int64_t cd = bsearch_idx<uint32_t>(mi[dm].insts, mi[dm].n_insts, H.col_gid[ms.col_off + c]);
              H.xmap.push_back((int32_t)cd);
            }
            for (uint32_t g = 0; g < mt.n_glob; ++g) {      // global rows: slot kept iff in P_src
              const uint32_t gid = H.grow_gid[mt.grow_off + g];
              int32_t src = -1;
              if (g < mt.n_stat) {                          // statics: same static visible in src
                src = (int32_t)bsearch_idx<uint32_t>(mi[sm].stats, mi[sm].n_stats, gid - (uint32_t)Lt);
              } else {                                      // heap: owner in Q_src, same ordinal
                const int32_t ct = H.grow_col[mt.grow_off + g];
                const uint32_t o = H.col_gid[mt.col_off + ct];
                int64_t cs = bsearch_idx<uint32_t>(mi[sm].insts, mi[sm].n_insts, o);
                if (cs >= 0) src = (int32_t)(H.col_hbase[ms.col_off + cs] + (g - H.col_hbase[mt.col_off + ct]));
              }
              H.xmap.push_back(src);
            }
          }
        }
      }
      const NodeRec& RS = H.nodes[nb + s];
      const uint32_t nch = n_chunks_of((uint32_t)(d->row_ptr[s + 1] - d->row_ptr[s]), RS.cls);
      if (RS.L > 0xffff) return set_err(GDROID_E_LIMIT, "app %u: method with > 65535 locals", k);
      Edge E{};
      E.dst = nb + s;
      E.info = (uint32_t)ek | ((uint32_t)RS.cls << 2) | ((nch - 1) << 5);
      E.off = RS.off; E.B = RS.B; E.L = (uint16_t)RS.L; E.logW = RS.logW;
      E.aux = (ek == GE_CALL) ? (int32_t)d->method_n_params[d->node_method[s]] : (ek == GE_RET ? RS.r0 : -1);
      E.xoff = xoff;
      H.edges.push_back(E);
    }
    if (kind == GK_CALL && n_c2r != 1) return set_err(GDROID_E_INVALID, "app %u: node %llu: a CALL needs exactly one C2R edge (V5)", k, (unsigned long long)n);
    H.row_ptr.push_back((uint32_t)H.edges.size());
  }
  for (uint64_t i = 0; i < d->n_entries; ++i) {
    if (d->entries[i] >= N || d->node_kind[d->entries[i]] != GK_ENTRY) return set_err(GDROID_E_INVALID, "app %u: entry %llu is not an ENTRY node", k, (unsigned long long)i);
    H.entries.push_back(nb + d->entries[i]);
  }
  return GDROID_OK;
}

size_t align256(size_t x) { return (x + 255) & ~size_t(255); }

}  // namespace

struct gdroid_app {
  int device = 0;
  cudaStream_t stream = nullptr;
  uint32_t n_apps = 0;
  std::vector<uint32_t> app_base;     // [n_apps+1] global node id ranges
  Dev D{};
  void* d_tables = nullptr;
  uint64_t* d_facts = nullptr;
  void* d_state = nullptr;            // stamp, queue, counts, stats, bar, digests
  DevStats* h_stats = nullptr;        // pinned
  uint64_t* d_scratch = nullptr;
  size_t scratch_bytes = 0;
  cudaEvent_t ev[4] = {nullptr, nullptr, nullptr, nullptr};
  gdroid_build_stats last{};
  uint64_t h2d_ns = 0;
  uint64_t launches = 0;
  bool built = false, pending = false;
  int max_blocks = 0;
};

namespace {

void free_app(gdroid_app* a) {
  if (!a) return;
  int cur = 0;
  cudaGetDevice(&cur);
  cudaSetDevice(a->device);
  if (a->d_tables) cudaFree(a->d_tables);
  if (a->d_facts) cudaFree(a->d_facts);
  if (a->d_state) cudaFree(a->d_state);
  if (a->d_scratch) cudaFree(a->d_scratch);
  if (a->D.trace) cudaFree(a->D.trace);
  if (a->h_stats) cudaFreeHost(a->h_stats);
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

gdroid_status ensure_scratch(gdroid_app* a, size_t bytes) {
  if (a->scratch_bytes >= bytes) return GDROID_OK;
  if (a->d_scratch) cudaFree(a->d_scratch);
  a->d_scratch = nullptr;
  a->scratch_bytes = 0;
  CU(cudaMalloc(&a->d_scratch, bytes));
  a->scratch_bytes = bytes;
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
  a->built = true;
  if (out) *out = s;
  if (h.limit_hit) return set_err(GDROID_E_LIMIT, "max_rounds (%u) exceeded; facts are an under-approximation", a->D.max_rounds);
  return GDROID_OK;
}

}  // namespace

extern "C" {

uint32_t gdroid_abi_version(void) { return GDROID_ABI_VERSION; }
const char* gdroid_last_error(void) { return g_err.c_str(); }

gdroid_status gdroid_load_batch(const gdroid_icfg_desc* descs, uint32_t n_apps, int device, void* cuda_stream,
                                gdroid_app** out) {
  if (!out) return set_err(GDROID_E_INVALID, "out is NULL");
  *out = nullptr;
  if (!descs || n_apps == 0 || n_apps > 65535) return set_err(GDROID_E_INVALID, "need 1..65535 apps");
  HostImage H;
  for (uint32_t k = 0; k < n_apps; ++k) {
    gdroid_status st = add_app(H, &descs[k], k);
    if (st != GDROID_OK) return st;
  }
  const uint32_t N = (uint32_t)H.nodes.size();
  const uint32_t n_entries = (uint32_t)H.entries.size();
  // work items: every node's out-edges in at most 32 chunks (queue entry = node << 5 | chunk)
  if (N >= (1u << 27)) return set_err(GDROID_E_LIMIT, "batch exceeds 2^27 nodes");
  uint64_t nc64 = 0;
  for (uint32_t n = 0; n < N; ++n) {
    const uint32_t c = n_chunks_of(H.nodes[n].e1 - H.nodes[n].e0, H.nodes[n].cls);
    H.cls_count[H.nodes[n].cls] += c;
    nc64 += c;
  }
  if (nc64 >= (1ull << 31)) return set_err(GDROID_E_LIMIT, "too many work items");
  const uint32_t NC = (uint32_t)nc64;
  H.app_node_base.push_back(N);
  if (H.tf.empty()) H.tf.push_back(0);          // keep every table non-empty
  if (H.xmap.empty()) H.xmap.push_back(-1);
  if (H.frow.empty()) H.frow.push_back(-1);
  if (H.args.empty()) H.args.push_back(-1);
  if (H.entries.empty()) H.entries.push_back(0);

  gdroid_app* a = new gdroid_app;
  a->device = device;
  a->stream = (cudaStream_t)cuda_stream;
  a->n_apps = n_apps;
  a->app_base = H.app_node_base;
  DeviceGuard guard(device);
  auto fail = [&](gdroid_status st) { free_app(a); return st; };

  // ---- one table buffer, uploaded from one pinned staging buffer
  struct Part { const void* src; size_t bytes; size_t off; };
  std::vector<Part> parts;
  size_t total = 0;
  auto add = [&](const void* p, size_t bytes) { parts.push_back({p, bytes, total}); total += align256(bytes); return parts.size() - 1; };
  size_t i_nodes = add(H.nodes.data(), H.nodes.size() * sizeof(NodeRec));
  size_t i_meths = add(H.meths.data(), H.meths.size() * sizeof(MethRec));
  size_t i_mods = add(H.mods.data(), H.mods.size() * sizeof(ModRec));
  size_t i_rp = add(H.row_ptr.data(), H.row_ptr.size() * 4);
  size_t i_e = add(H.edges.data(), H.edges.size() * sizeof(Edge));
  size_t i_ap = add(H.arg_ptr.data(), H.arg_ptr.size() * 4);
  size_t i_a = add(H.args.data(), H.args.size() * 4);
  size_t i_cg = add(H.col_gid.data(), H.col_gid.size() * 4);
  size_t i_ct = add(H.col_type.data(), H.col_type.size() * 4);
  size_t i_ch = add(H.col_hbase.data(), H.col_hbase.size() * 4);
  size_t i_gg = add(H.grow_gid.data(), H.grow_gid.size() * 4);
  size_t i_gc = add(H.grow_col.data(), H.grow_col.size() * 4);
  size_t i_gf = add(H.grow_field.data(), H.grow_field.size() * 4);
  size_t i_tp = add(H.tf_ptr.data(), H.tf_ptr.size() * 4);
  size_t i_tf = add(H.tf.data(), H.tf.size() * 4);
  size_t i_xm = add(H.xmap.data(), H.xmap.size() * 4);
  size_t i_nb = add(H.app_node_base.data(), H.app_node_base.size() * 4);
  size_t i_en = add(H.entries.data(), H.entries.size() * 4);
  size_t i_nm = add(H.node_method.data(), H.node_method.size() * 4);
  size_t i_fr = add(H.frow.data(), H.frow.size() * 4);

  auto t0 = std::chrono::steady_clock::now();
  {
    cudaError_t e = cudaMalloc(&a->d_tables, total);
    if (e != cudaSuccess) return fail(set_err(e == cudaErrorMemoryAllocation ? GDROID_E_OOM : GDROID_E_CUDA, "device tables (%zu B): %s", total, cudaGetErrorString(e)));
    void* stage = nullptr;
    e = cudaMallocHost(&stage, total);
    if (e != cudaSuccess) return fail(set_err(GDROID_E_OOM, "pinned staging (%zu B): %s", total, cudaGetErrorString(e)));
    for (auto& p : parts) if (p.bytes) std::memcpy((char*)stage + p.off, p.src, p.bytes);
    e = cudaMemcpyAsync(a->d_tables, stage, total, cudaMemcpyHostToDevice, a->stream);
    cudaError_t e2 = cudaStreamSynchronize(a->stream);
    cudaFreeHost(stage);
    if (e != cudaSuccess || e2 != cudaSuccess) return fail(set_err(GDROID_E_CUDA, "H2D upload: %s", cudaGetErrorString(e != cudaSuccess ? e : e2)));
  }
  a->h2d_ns = (uint64_t)std::chrono::duration_cast<std::chrono::nanoseconds>(std::chrono::steady_clock::now() - t0).count();
  char* T = (char*)a->d_tables;
  Dev& D = a->D;
  D.nodes = (const NodeRec*)(T + parts[i_nodes].off);
  D.meths = (const MethRec*)(T + parts[i_meths].off);
  D.mods = (const ModRec*)(T + parts[i_mods].off);
  D.row_ptr = (const uint32_t*)(T + parts[i_rp].off);
  D.edges = (const Edge*)(T + parts[i_e].off);
  D.arg_ptr = (const uint32_t*)(T + parts[i_ap].off);
  D.args = (const int32_t*)(T + parts[i_a].off);
  D.col_gid = (const uint32_t*)(T + parts[i_cg].off);
  D.col_type = (const int32_t*)(T + parts[i_ct].off);
  D.col_hbase = (const uint32_t*)(T + parts[i_ch].off);
  D.grow_gid = (const uint32_t*)(T + parts[i_gg].off);
  D.grow_col = (const int32_t*)(T + parts[i_gc].off);
  D.grow_field = (const int32_t*)(T + parts[i_gf].off);
  D.tf_ptr = (const uint32_t*)(T + parts[i_tp].off);
  D.tf = (const uint32_t*)(T + parts[i_tf].off);
  D.xmap = (const int32_t*)(T + parts[i_xm].off);
  D.app_node_base = (const uint32_t*)(T + parts[i_nb].off);
  D.entries = (const uint32_t*)(T + parts[i_en].off);
  D.node_method = (const uint32_t*)(T + parts[i_nm].off);
  D.frow = (const int32_t*)(T + parts[i_fr].off);
  D.n_nodes = N;
  D.n_chunks = NC;
  D.n_entries = n_entries;
  uint32_t acc = 0;
  for (int c = 0; c < NCLS; ++c) { D.seg[c] = acc; acc += H.cls_count[c]; }
  D.seg[NCLS] = acc;
  D.n_words = H.fact_words;

  // ---- fact store + mutable state
  {
    cudaError_t e = cudaMalloc(&a->d_facts, std::max<uint64_t>(H.fact_words, 4) * 8);
    if (e != cudaSuccess) return fail(set_err(GDROID_E_OOM, "fact store (%llu B): %s", (unsigned long long)(H.fact_words * 8), cudaGetErrorString(e)));
    D.facts = a->d_facts;
    size_t s_stamp = align256((size_t)N * 4), s_queue = align256((size_t)3 * NC * 4), s_counts = align256(3 * CNT_STRIDE * 4);
    size_t s_stats = align256(sizeof(DevStats)), s_bar = 256, s_nd = align256((size_t)N * 8), s_ad = align256((size_t)n_apps * 8);
    size_t st = s_stamp + s_queue + s_counts + s_stats + s_bar + s_nd + s_ad;
    e = cudaMalloc(&a->d_state, st);
    if (e != cudaSuccess) return fail(set_err(GDROID_E_OOM, "device state (%zu B): %s", st, cudaGetErrorString(e)));
    char* S = (char*)a->d_state;
    D.stamp = (uint32_t*)S; S += s_stamp;
    D.queue = (uint32_t*)S; S += s_queue;
    D.counts = (uint32_t*)S; S += s_counts;
    D.stats = (DevStats*)S; S += s_stats;
    D.bar = (uint32_t*)S; S += s_bar;
    D.node_digest = (uint64_t*)S; S += s_nd;
    D.app_digest = (unsigned long long*)S;
    e = cudaMallocHost(&a->h_stats, sizeof(DevStats));
    if (e != cudaSuccess) return fail(set_err(GDROID_E_OOM, "pinned stats: %s", cudaGetErrorString(e)));
    for (auto& ev : a->ev)
      if (cudaEventCreate(&ev) != cudaSuccess) return fail(set_err(GDROID_E_CUDA, "cudaEventCreate failed"));
  }
  a->max_blocks = fixpoint_max_blocks(device);
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
  cudaStream_t s = a->stream;
  const uint32_t N = D.n_nodes;
  uint32_t blocks = o.blocks ? std::min<uint32_t>(o.blocks, (uint32_t)a->max_blocks) : (uint32_t)a->max_blocks;
  a->launches = 0;
  CU(cudaEventRecord(a->ev[0], s));
  // (a2) zero the fact matrices and the worklist state
  CU(cudaMemsetAsync(D.facts, 0, D.n_words * 8, s));
  CU(cudaMemsetAsync(D.stamp, 0, (size_t)N * 4, s));
  CU(cudaMemsetAsync(D.counts, 0, 3 * CNT_STRIDE * 4, s));
  CU(cudaMemsetAsync(D.stats, 0, sizeof(DevStats), s));
  CU(cudaMemsetAsync(D.bar, 0, 16, s));
  CU(cudaMemsetAsync(D.app_digest, 0, (size_t)a->n_apps * 8, s));
  CU(launch_seed(D, s));
  a->launches++;
  CU(cudaEventRecord(a->ev[1], s));
  if (o.loop_mode == 0) {
    CU(launch_fixpoint(D, blocks, s));
    a->launches++;
  } else {
    // one launch per round; the host looks ahead K rounds between termination checks
    const uint32_t K = 64;
    uint32_t* h_counts = nullptr;
    CU(cudaMallocHost(&h_counts, 3 * CNT_STRIDE * 4 + 16));
    uint32_t round = 1;
    for (;;) {
      for (uint32_t q = 0; q < K; ++q) {
        cudaError_t e = launch_round(D, round + q, blocks, s);
        if (e != cudaSuccess) { cudaFreeHost(h_counts); return set_err(GDROID_E_CUDA, "k_round: %s", cudaGetErrorString(e)); }
        a->launches++;
      }
      round += K;
      cudaMemcpyAsync(h_counts, D.bar, 16, cudaMemcpyDeviceToHost, s);
      cudaError_t e = cudaStreamSynchronize(s);
      if (e != cudaSuccess) { cudaFreeHost(h_counts); return set_err(GDROID_E_CUDA, "round loop: %s", cudaGetErrorString(e)); }
      if (h_counts[2]) break;                                      // a round found an empty worklist
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
  CU(launch_popc(a->D, n0, n1, a->d_scratch, a->stream));
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
  CU(launch_expand(a->D, n0, n1, d_ptr, d_pairs, a->stream));
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
  CU(launch_popc(a->D, g, g + 1, a->d_scratch, a->stream));
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
  CU(launch_expand(a->D, g, g + 1, a->d_scratch, a->d_scratch + 2, a->stream));
  CU(cudaMemcpyAsync(pairs, a->d_scratch + 2, (size_t)cnt * 8, cudaMemcpyDeviceToHost, a->stream));
  CU(cudaStreamSynchronize(a->stream));
  return GDROID_OK;
}

gdroid_status gdroid_read_facts(const gdroid_app* a, uint32_t node, uint64_t* pairs, uint64_t cap, uint64_t* n_pairs) {
  return gdroid_read_facts_in(a, 0, node, pairs, cap, n_pairs);
}

gdroid_status gdroid_node_digests(const gdroid_app* ca, uint64_t* per_node, uint64_t* app_digest) {
  gdroid_app* a = const_cast<gdroid_app*>(ca);
  if (!a) return set_err(GDROID_E_INVALID, "app is NULL");
  if (!a->built) return set_err(GDROID_E_STATE, "digests read before a completed build");
  DeviceGuard guard(a->device);
  const uint32_t n = a->app_base[1] - a->app_base[0];
  if (per_node) CU(cudaMemcpyAsync(per_node, a->D.node_digest, (size_t)n * 8, cudaMemcpyDeviceToHost, a->stream));
  if (app_digest) CU(cudaMemcpyAsync(app_digest, a->D.app_digest, 8, cudaMemcpyDeviceToHost, a->stream));
  CU(cudaStreamSynchronize(a->stream));
  return GDROID_OK;
}

gdroid_status gdroid_app_digests(const gdroid_app* ca, uint64_t* per_app) {
  gdroid_app* a = const_cast<gdroid_app*>(ca);
  if (!a || !per_app) return set_err(GDROID_E_INVALID, "NULL argument");
  if (!a->built) return set_err(GDROID_E_STATE, "digests read before a completed build");
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
