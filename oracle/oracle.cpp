// oracle.cpp — plain, slow, single-threaded CPU oracle for GDroid's IDFG construction.
//
// TEST INFRASTRUCTURE ONLY (see oracle.h).  Shares no code with the CUDA path.
//
// Facts are explicit sorted std::vector<uint64_t> sets of (slot_gid << 32 | inst_gid)
// pairs — the paper's set-based representation (Fig. 5a), NOT bitsets.
// Each function cites the passage (or SURVEY.md §8(c) reading, restated in DESIGN.md §3)
// it follows.  Pins: tests/test_oracle_*.py (golden tiny, Fig. 2 rounds, Fig. 7 merge,
// Kleene brute force, Andersen / reaching-definitions reductions, inlining law).
#include "oracle.h"

#include <algorithm>
#include <chrono>
#include <cstdio>
#include <cstring>
#include <deque>
#include <queue>
#include <functional>
#include <string>
#include <vector>

namespace {

typedef std::vector<uint64_t> PairSet;  // sorted, unique

enum { NOP, ENTRY, EXIT, RETSITE, CALL, PRIM, CONST, NEW, COPY, SLOAD, SSTORE, RETV,
       FLOAD, FSTORE, ALOAD, ASTORE, N_KINDS };
enum { E_INTRA, E_CALL, E_RET, E_C2R };
const uint32_t F_ARR = 0;

thread_local std::string g_err;

int fail(int code, const char* fmt, long long a = 0, long long b = 0) {
  char buf[512];
  snprintf(buf, sizeof buf, fmt, a, b);
  g_err = buf;
  return code;
}

inline uint64_t pack(uint64_t s, uint64_t o) { return (s << 32) | o; }
inline uint32_t slot_of(uint64_t p) { return (uint32_t)(p >> 32); }
inline uint32_t inst_of(uint64_t p) { return (uint32_t)(p & 0xffffffffu); }

// splitmix64 finaliser
inline uint64_t mix64(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ULL;
  z = (z ^ (z >> 27)) * 0x94d049bb133111ebULL;
  return z ^ (z >> 31);
}

// Universe bookkeeping: slot numbering of SURVEY §8(b) (locals, statics, heap slots).
struct Universe {
  const oracle_icfg* g;
  std::vector<uint64_t> local_base;  // [M+1]
  uint64_t L_total = 0, G = 0;
  std::vector<uint64_t> heap_base;  // [I+1]  heap slots of instance o: [heap_base[o], heap_base[o+1])
  std::vector<std::vector<char>> mod_has_inst;    // per module, per instance gid
  std::vector<std::vector<char>> mod_has_static;  // per module, per static index

  void init(const oracle_icfg* gg) {
    g = gg;
    local_base.assign(g->n_methods + 1, 0);
    for (uint32_t m = 0; m < g->n_methods; ++m) local_base[m + 1] = local_base[m] + g->method_n_locals[m];
    L_total = local_base[g->n_methods];
    G = g->n_statics;
    heap_base.assign(g->n_instances + 1, 0);
    for (uint32_t o = 0; o < g->n_instances; ++o) {
      int32_t t = g->inst_type[o];
      uint64_t nf = (t < 0) ? 0 : (g->type_field_ptr[t + 1] - g->type_field_ptr[t]);
      heap_base[o + 1] = heap_base[o] + nf;
    }
    mod_has_inst.assign(g->n_modules, std::vector<char>(g->n_instances, 0));
    mod_has_static.assign(g->n_modules, std::vector<char>(g->n_statics, 0));
    for (uint32_t d = 0; d < g->n_modules; ++d) {
      for (uint64_t k = g->module_inst_ptr[d]; k < g->module_inst_ptr[d + 1]; ++k)
        mod_has_inst[d][g->module_insts[k]] = 1;
      for (uint64_t k = g->module_static_ptr[d]; k < g->module_static_ptr[d + 1]; ++k)
        mod_has_static[d][g->module_statics[k]] = 1;
    }
  }
  bool is_local(uint64_t s) const { return s < L_total; }
  bool is_global(uint64_t s) const { return s >= L_total; }
  bool is_local_of(uint64_t s, uint32_t m) const { return s >= local_base[m] && s < local_base[m + 1]; }
  uint64_t ret_slot(uint32_t m) const { return local_base[m + 1] - 1; }
  uint64_t param_slot(uint32_t m, uint32_t j) const { return local_base[m] + j; }
  // heap slot (o, f): exists iff o != NULL and f in F(t(o))  (C1)
  int64_t heap_slot(uint32_t o, uint32_t f) const {
    int32_t t = g->inst_type[o];
    if (t < 0) return -1;
    for (uint64_t k = g->type_field_ptr[t]; k < g->type_field_ptr[t + 1]; ++k)
      if (g->type_fields[k] == f) return (int64_t)(L_total + G + heap_base[o] + (k - g->type_field_ptr[t]));
    return -1;
  }
  // instance owning heap slot s (s must be a heap slot)
  uint32_t heap_owner(uint64_t s) const {
    uint64_t h = s - L_total - G;
    return (uint32_t)(std::upper_bound(heap_base.begin(), heap_base.end(), h) - heap_base.begin() - 1);
  }
  // π_m membership (C1): slot s ∈ P_m and instance o ∈ Q_m
  bool in_pool(uint32_t m, uint64_t s, uint32_t o) const {
    uint32_t d = g->method_module[m];
    if (!mod_has_inst[d][o]) return false;
    if (s < L_total) return is_local_of(s, m);
    if (s < L_total + G) return mod_has_static[d][s - L_total] != 0;
    return mod_has_inst[d][heap_owner(s)] != 0;
  }
};

// instances o with (s, o) ∈ X, ascending
void pts(const PairSet& X, uint64_t s, std::vector<uint32_t>& out) {
  out.clear();
  auto it = std::lower_bound(X.begin(), X.end(), pack(s, 0));
  for (; it != X.end() && slot_of(*it) == s; ++it) out.push_back(inst_of(*it));
}

bool contains(const PairSet& X, uint64_t p) { return std::binary_search(X.begin(), X.end(), p); }

// X \ K(v)   (K(v) = {(v,o) : o ∈ Inst}, C2)
PairSet kill(const PairSet& X, uint64_t v) {
  PairSet Y;
  Y.reserve(X.size());
  for (uint64_t p : X)
    if (slot_of(p) != v) Y.push_back(p);
  return Y;
}

void normalize(PairSet& Z) {
  std::sort(Z.begin(), Z.end());
  Z.erase(std::unique(Z.begin(), Z.end()), Z.end());
}

PairSet set_union(const PairSet& A, const PairSet& B) {
  PairSet C;
  C.reserve(A.size() + B.size());
  std::set_union(A.begin(), A.end(), B.begin(), B.end(), std::back_inserter(C));
  return C;
}

// ---------------------------------------------------------------------------------------
// Node transfer functions f_n(X) — SURVEY §8(c) C2 table (readings A2, A3, A8, A23).
// GEN is evaluated on X before the kill.
// ---------------------------------------------------------------------------------------
PairSet transfer(const Universe& U, uint32_t n, const PairSet& X) {
  const oracle_icfg* g = U.g;
  const int32_t* op = g->node_ops + 4ull * n;
  uint32_t m = g->node_method[n];
  std::vector<uint32_t> tmp, tmp2;
  PairSet gen;
  switch (g->node_kind[n]) {
    case NOP: case ENTRY: case EXIT: case RETSITE: case CALL:
      return X;                                                   // f(X) = X
    case PRIM:
      return kill(X, (uint64_t)op[0]);                             // X \ K(v)
    case CONST: case NEW:
      gen.push_back(pack((uint64_t)op[0], (uint32_t)op[3]));       // (X \ K(v)) ∪ {(v,o_n)}
      return set_union(kill(X, (uint64_t)op[0]), gen);
    case COPY: case SLOAD: {                                       // (X \ K(v)) ∪ {(v,o):(w,o)∈X}
      pts(X, (uint64_t)op[1], tmp);
      for (uint32_t o : tmp) gen.push_back(pack((uint64_t)op[0], o));
      return set_union(kill(X, (uint64_t)op[0]), gen);
    }
    case SSTORE: {                                                 // X ∪ {(g,o):(w,o)∈X} (weak)
      pts(X, (uint64_t)op[1], tmp);
      for (uint32_t o : tmp) gen.push_back(pack((uint64_t)op[0], o));
      return set_union(X, gen);
    }
    case RETV: {                                                   // (X \ K(RET_m)) ∪ {(RET_m,o):(w,o)∈X}
      uint64_t r = U.ret_slot(m);
      pts(X, (uint64_t)op[1], tmp);
      for (uint32_t o : tmp) gen.push_back(pack(r, o));
      return set_union(kill(X, r), gen);
    }
    case FLOAD: case ALOAD: {                                      // v = w.f
      uint32_t f = (g->node_kind[n] == ALOAD) ? F_ARR : (uint32_t)op[2];
      pts(X, (uint64_t)op[1], tmp);
      for (uint32_t o1 : tmp) {
        if (o1 == 0) continue;                                     // NULL has no fields (A23)
        int64_t hs = U.heap_slot(o1, f);
        if (hs < 0) continue;                                      // f ∉ F(t(o1))
        pts(X, (uint64_t)hs, tmp2);
        for (uint32_t o2 : tmp2) gen.push_back(pack((uint64_t)op[0], o2));
      }
      normalize(gen);
      return set_union(kill(X, (uint64_t)op[0]), gen);
    }
    case FSTORE: case ASTORE: {                                    // v.f = w  (weak)
      uint32_t f = (g->node_kind[n] == ASTORE) ? F_ARR : (uint32_t)op[2];
      pts(X, (uint64_t)op[0], tmp);
      pts(X, (uint64_t)op[1], tmp2);
      for (uint32_t o1 : tmp) {
        if (o1 == 0) continue;
        int64_t hs = U.heap_slot(o1, f);
        if (hs < 0) continue;
        for (uint32_t o2 : tmp2) gen.push_back(pack((uint64_t)hs, o2));
      }
      normalize(gen);
      return set_union(X, gen);
    }
  }
  return X;
}

// ---------------------------------------------------------------------------------------
// Edge transforms T_e(Y) — SURVEY §8(c) C3 (readings A7, A9).
// ---------------------------------------------------------------------------------------
PairSet edge_transform(const Universe& U, uint32_t p, uint32_t s, uint8_t kind, const PairSet& Y) {
  const oracle_icfg* g = U.g;
  PairSet Z;
  switch (kind) {
    case E_INTRA:
      return Y;
    case E_CALL: {   // π_{m'}({(param_j(m'),o) : (arg_j(c),o) ∈ Y} ∪ Glob(Y))
      uint32_t callee = g->node_method[s];
      std::vector<uint32_t> tmp;
      uint64_t a0 = g->call_arg_ptr[p], a1 = g->call_arg_ptr[p + 1];
      for (uint64_t j = 0; j < a1 - a0; ++j) {
        int32_t arg = g->call_args[a0 + j];
        if (arg < 0) continue;                                     // non-reference actual
        pts(Y, (uint64_t)arg, tmp);
        for (uint32_t o : tmp) Z.push_back(pack(U.param_slot(callee, (uint32_t)j), o));
      }
      for (uint64_t q : Y)
        if (U.is_global(slot_of(q))) Z.push_back(q);
      normalize(Z);
      PairSet W;
      for (uint64_t q : Z)
        if (U.in_pool(callee, slot_of(q), inst_of(q))) W.push_back(q);
      return W;
    }
    case E_C2R: {    // {(s,o) ∈ Y : s ∈ locals(m(c)), s ≠ lhs(c)} ∪ Glob(Y)
      uint32_t m = g->node_method[p];
      int32_t lhs = g->node_ops[4ull * p + 0];
      for (uint64_t q : Y) {
        uint64_t sl = slot_of(q);
        if (U.is_global(sl) || (U.is_local_of(sl, m) && (lhs < 0 || sl != (uint64_t)lhs))) Z.push_back(q);
      }
      return Z;
    }
    case E_RET: {    // π_{m(c)}({(lhs(c),o) : (RET_{m'},o) ∈ Y} ∪ Glob(Y))
      uint32_t callee = g->node_method[p];
      uint32_t caller = g->node_method[s];
      int32_t lhs = g->node_ops[4ull * s + 0];                     // RETSITE carries lhs(c)
      std::vector<uint32_t> tmp;
      if (lhs >= 0) {
        pts(Y, U.ret_slot(callee), tmp);
        for (uint32_t o : tmp) Z.push_back(pack((uint64_t)lhs, o));
      }
      for (uint64_t q : Y)
        if (U.is_global(slot_of(q))) Z.push_back(q);
      normalize(Z);
      PairSet W;
      for (uint64_t q : Z)
        if (U.in_pool(caller, slot_of(q), inst_of(q))) W.push_back(q);
      return W;
    }
  }
  return Z;
}

// IN[s] := IN[s] ∪ Z ; returns whether IN[s] grew (A6)
bool merge_union(PairSet& IN, const PairSet& Z) {
  if (Z.empty()) return false;
  PairSet C = set_union(IN, Z);
  bool grew = C.size() != IN.size();
#ifdef ORACLE_DEBUG
  if (!std::includes(C.begin(), C.end(), IN.begin(), IN.end())) abort();  // monotone
#endif
  IN.swap(C);
  return grew;
}

// ---------------------------------------------------------------------------------------
// Validation V1-V6.
// ---------------------------------------------------------------------------------------
int validate(const Universe& U) {
  const oracle_icfg* g = U.g;
  const uint64_t N = g->n_nodes;
  if (g->row_ptr[0] != 0) return fail(-1, "row_ptr[0] != 0");
  for (uint64_t n = 0; n < N; ++n)
    if (g->row_ptr[n + 1] < g->row_ptr[n]) return fail(-1, "row_ptr not monotone at %lld", (long long)n);
  if (g->row_ptr[N] != g->n_edges) return fail(-1, "row_ptr[N] != n_edges");
  for (uint32_t m = 0; m < g->n_methods; ++m) {
    if (g->method_module[m] >= g->n_modules) return fail(-1, "method %lld module out of range", m);
    if (g->method_n_locals[m] < g->method_n_params[m] + 1) return fail(-1, "method %lld: n_locals < n_params+1", m);
    if (g->method_entry[m] >= N || g->node_kind[g->method_entry[m]] != ENTRY) return fail(-1, "method %lld entry", m);
    if (g->method_exit[m] >= N || g->node_kind[g->method_exit[m]] != EXIT) return fail(-1, "method %lld exit", m);
  }
  for (uint32_t d = 0; d < g->n_modules; ++d) {
    if (!U.mod_has_inst[d][0]) return fail(-2, "module %lld pool lacks NULL", d);
  }
  if (g->inst_type[0] != -1) return fail(-1, "instance 0 must be NULL (type -1)");
  for (uint64_t n = 0; n < N; ++n) {
    uint32_t k = g->node_kind[n], m = g->node_method[n];
    if (k >= N_KINDS) return fail(-1, "node %lld: bad kind", (long long)n);
    if (m >= g->n_methods) return fail(-1, "node %lld: method out of range", (long long)n);
    uint32_t d = g->method_module[m];
    const int32_t* op = g->node_ops + 4 * n;
    auto local_ok = [&](int32_t s) { return s >= 0 && U.is_local_of((uint64_t)s, m); };
    auto static_ok = [&](int32_t s) {
      return s >= 0 && (uint64_t)s >= U.L_total && (uint64_t)s < U.L_total + U.G;
    };
    switch (k) {
      case PRIM: if (!local_ok(op[0])) return fail(-2, "node %lld: lhs not a local of its method (V4)", (long long)n); break;
      case CONST: case NEW:
        if (!local_ok(op[0])) return fail(-2, "node %lld: lhs not a local of its method (V4)", (long long)n);
        if (op[3] < 0 || (uint32_t)op[3] >= g->n_instances) return fail(-1, "node %lld: instance out of range", (long long)n);
        if (k == NEW && op[3] == 0) return fail(-1, "node %lld: NEW of NULL", (long long)n);
        if (!U.mod_has_inst[d][op[3]]) return fail(-2, "node %lld: site instance not in module pool (V1)", (long long)n);
        break;
      case COPY: case FLOAD: case FSTORE: case ALOAD: case ASTORE:
        if (!local_ok(op[0]) || !local_ok(op[1])) return fail(-2, "node %lld: operand not a local of its method (V4)", (long long)n);
        if ((k == FLOAD || k == FSTORE) && (op[2] < 0 || (uint32_t)op[2] >= g->n_fields)) return fail(-1, "node %lld: field out of range", (long long)n);
        break;
      case SLOAD:
        if (!local_ok(op[0])) return fail(-2, "node %lld: lhs not a local (V4)", (long long)n);
        if (!static_ok(op[1])) return fail(-1, "node %lld: rhs not a static slot", (long long)n);
        if (!U.mod_has_static[d][op[1] - U.L_total]) return fail(-2, "node %lld: static not visible in module (V2)", (long long)n);
        break;
      case SSTORE:
        if (!local_ok(op[1])) return fail(-2, "node %lld: rhs not a local (V4)", (long long)n);
        if (!static_ok(op[0])) return fail(-1, "node %lld: lhs not a static slot", (long long)n);
        if (!U.mod_has_static[d][op[0] - U.L_total]) return fail(-2, "node %lld: static not visible in module (V2)", (long long)n);
        break;
      case RETV:
        if (!local_ok(op[1])) return fail(-2, "node %lld: rhs not a local (V4)", (long long)n);
        break;
      case CALL:
        if (op[0] >= 0 && !local_ok(op[0])) return fail(-2, "node %lld: call lhs not a local (V4)", (long long)n);
        for (uint64_t a = g->call_arg_ptr[n]; a < g->call_arg_ptr[n + 1]; ++a)
          if (g->call_args[a] >= 0 && !local_ok(g->call_args[a])) return fail(-2, "node %lld: arg not a local (V4)", (long long)n);
        break;
      case RETSITE: {
        if (op[3] < 0 || (uint64_t)op[3] >= N || g->node_kind[op[3]] != CALL) return fail(-1, "node %lld: RETSITE without CALL", (long long)n);
        if (g->node_method[op[3]] != m || g->node_ops[4ull * op[3]] != op[0]) return fail(-1, "node %lld: RETSITE/CALL mismatch", (long long)n);
        break;
      }
      default: break;
    }
    if (k != CALL && g->call_arg_ptr[n + 1] != g->call_arg_ptr[n]) return fail(-1, "node %lld: args on non-CALL", (long long)n);
    // edges (V5, V6)
    int n_c2r = 0;
    for (uint64_t e = g->row_ptr[n]; e < g->row_ptr[n + 1]; ++e) {
      uint32_t s = g->col[e];
      if (s >= N) return fail(-1, "edge %lld: target out of range", (long long)e);
      switch (g->edge_kind[e]) {
        case E_INTRA:
          if (k == CALL || k == EXIT || g->node_method[s] != m) return fail(-1, "edge %lld: bad INTRA edge (V5)", (long long)e);
          break;
        case E_CALL: {
          if (k != CALL || g->node_kind[s] != ENTRY) return fail(-1, "edge %lld: bad CALL edge (V5)", (long long)e);
          uint32_t callee = g->node_method[s];
          if (g->method_entry[callee] != s) return fail(-1, "edge %lld: CALL target not a method entry", (long long)e);
          if (g->call_arg_ptr[n + 1] - g->call_arg_ptr[n] != g->method_n_params[callee])
            return fail(-1, "edge %lld: arity mismatch (V6)", (long long)e);
          break;
        }
        case E_C2R:
          if (k != CALL || g->node_kind[s] != RETSITE || (uint32_t)g->node_ops[4ull * s + 3] != n)
            return fail(-1, "edge %lld: bad C2R edge (V5)", (long long)e);
          ++n_c2r;
          break;
        case E_RET: {
          if (k != EXIT || g->node_kind[s] != RETSITE) return fail(-1, "edge %lld: bad RET edge (V5)", (long long)e);
          uint32_t c = (uint32_t)g->node_ops[4ull * s + 3];
          bool ok = false;
          for (uint64_t e2 = g->row_ptr[c]; e2 < g->row_ptr[c + 1]; ++e2)
            if (g->edge_kind[e2] == E_CALL && g->col[e2] == g->method_entry[m]) ok = true;
          if (!ok) return fail(-1, "edge %lld: RET to a site that does not call this method (V5)", (long long)e);
          break;
        }
        default: return fail(-1, "edge %lld: bad edge kind", (long long)e);
      }
    }
    if (k == CALL && n_c2r != 1) return fail(-1, "node %lld: CALL needs exactly one C2R edge (V5)", (long long)n);
  }
  for (uint32_t i = 0; i < g->n_entries; ++i)
    if (g->entries[i] >= N || g->node_kind[g->entries[i]] != ENTRY) return fail(-1, "entry %lld not an ENTRY node", i);
  return 0;
}

}  // namespace

struct oracle_result {
  std::vector<PairSet> IN;
  std::vector<char> visited;
  uint64_t visits = 0;
  double seconds = 0;
};

extern "C" {

const char* oracle_last_error(void) { return g_err.c_str(); }

// Alg. 1 IDFGBuilding with readings A4 (fact = IN), A5 (first-reach),
// A6 (update = grew): SURVEY §8(c) C5.
int oracle_build(const oracle_icfg* g, int order, uint64_t seed, oracle_result** out) {
  *out = nullptr;
  Universe U;
  U.init(g);
  int rc = validate(U);
  if (rc) return rc;
  auto t0 = std::chrono::steady_clock::now();
  oracle_result* R = new oracle_result;
  const uint32_t N = g->n_nodes;
  R->IN.assign(N, PairSet());                  // l.5-7: an empty set per node
  R->visited.assign(N, 0);
  std::vector<char> in_wl(N, 0);
  std::deque<uint32_t> wl;                     // l.8
  std::priority_queue<uint32_t, std::vector<uint32_t>, std::greater<uint32_t>> pq;   // order 3
  auto push = [&](uint32_t x) { if (order == 3) pq.push(x); else wl.push_back(x); in_wl[x] = 1; };
  for (uint32_t i = 0; i < g->n_entries; ++i)  // l.9: worklist <- entry
    if (!in_wl[g->entries[i]]) push(g->entries[i]);
  uint64_t rng = seed * 0x9e3779b97f4a7c15ULL + 1;
  while (!wl.empty() || !pq.empty()) {         // l.10
    uint32_t n;
    if (order == 3) { n = pq.top(); pq.pop(); }
    else if (order == 1) { n = wl.back(); wl.pop_back(); }
    else if (order == 2) {
      rng ^= rng << 13; rng ^= rng >> 7; rng ^= rng << 17;
      size_t i = (size_t)(rng % wl.size());
      n = wl[i]; wl[i] = wl.back(); wl.pop_back();
    } else { n = wl.front(); wl.pop_front(); }  // l.11-12
    in_wl[n] = 0;
    R->visited[n] = 1;
    ++R->visits;
    PairSet Y = transfer(U, n, R->IN[n]);      // ProcessNode: GEN_KILL
    for (uint64_t e = g->row_ptr[n]; e < g->row_ptr[n + 1]; ++e) {  // SEARCH
      uint32_t s = g->col[e];
      PairSet Z = edge_transform(U, n, s, g->edge_kind[e], Y);
      bool grew = merge_union(R->IN[s], Z);    // union + update()
      if ((grew || !R->visited[s]) && !in_wl[s]) push(s);  // l.13-14
    }
  }
  R->seconds = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
  *out = R;
  return 0;
}

void oracle_free(oracle_result* r) { delete r; }
uint64_t oracle_visits(const oracle_result* r) { return r->visits; }
double oracle_seconds(const oracle_result* r) { return r->seconds; }
uint64_t oracle_total_pairs(const oracle_result* r) {
  uint64_t t = 0;
  for (auto& s : r->IN) t += s.size();
  return t;
}
void oracle_all_pairs(const oracle_result* r, uint64_t* ptr, uint64_t* pairs) {
  uint64_t k = 0;
  for (size_t n = 0; n < r->IN.size(); ++n) {
    if (ptr) ptr[n] = k;
    if (pairs) std::memcpy(pairs + k, r->IN[n].data(), r->IN[n].size() * 8);
    k += r->IN[n].size();
  }
  if (ptr) ptr[r->IN.size()] = k;
}

// C8: d(n) = Σ_{(s,o)∈IN(n)} mix64(mix64(n) ^ ((s<<32)|o)) mod 2^64 ; app = Σ_n d(n)
void oracle_digests(const oracle_result* r, uint64_t* per_node, uint64_t* app) {
  uint64_t a = 0;
  for (size_t n = 0; n < r->IN.size(); ++n) {
    uint64_t hn = mix64((uint64_t)n), d = 0;
    for (uint64_t p : r->IN[n]) d += mix64(hn ^ p);
    if (per_node) per_node[n] = d;
    a += d;
  }
  if (app) *app = a;
}

uint64_t oracle_check_postfix(const oracle_icfg* g, const oracle_result* r) {
  Universe U;
  U.init(g);
  uint64_t bad = 0;
  for (uint32_t p = 0; p < g->n_nodes; ++p) {
    if (!r->visited[p]) { bad += r->IN[p].empty() ? 0 : 1; continue; }
    PairSet Y = transfer(U, p, r->IN[p]);
    for (uint64_t e = g->row_ptr[p]; e < g->row_ptr[p + 1]; ++e) {
      uint32_t s = g->col[e];
      PairSet Z = edge_transform(U, p, s, g->edge_kind[e], Y);
      for (uint64_t q : Z) bad += contains(r->IN[s], q) ? 0 : 1;
      if (!r->visited[s]) ++bad;   // every successor of a reached node is reached
    }
  }
  return bad;
}

// Round-synchronous (BSP) variant of Alg. 1 for the Fig. 2 pin (reading A12): every round
// processes the whole current list in order; successors that grew or were never reached (A5)
// form the next list, each once.  Same fixed point as the FIFO worklist.
int64_t oracle_bsp_rounds(const oracle_icfg* g, uint32_t* seq, uint64_t cap, uint32_t* lens, uint64_t lens_cap) {
  Universe U;
  U.init(g);
  int rc = validate(U);
  if (rc) return rc;
  const uint32_t N = g->n_nodes;
  std::vector<PairSet> IN(N);
  std::vector<char> visited(N, 0), in_next(N, 0);
  std::vector<uint32_t> cur, nxt;
  for (uint32_t i = 0; i < g->n_entries; ++i)
    if (std::find(cur.begin(), cur.end(), g->entries[i]) == cur.end()) cur.push_back(g->entries[i]);
  uint64_t k = 0;
  int64_t rounds = 0;
  while (!cur.empty()) {
    if ((uint64_t)rounds < lens_cap) lens[rounds] = (uint32_t)cur.size();
    for (uint32_t n : cur) { if (k < cap) seq[k] = n; ++k; }
    ++rounds;
    nxt.clear();
    for (uint32_t n : cur) {
      visited[n] = 1;
      PairSet Y = transfer(U, n, IN[n]);
      for (uint64_t e = g->row_ptr[n]; e < g->row_ptr[n + 1]; ++e) {
        uint32_t s = g->col[e];
        PairSet Z = edge_transform(U, n, s, g->edge_kind[e], Y);
        bool grew = merge_union(IN[s], Z);
        if ((grew || !visited[s]) && !in_next[s]) { nxt.push_back(s); in_next[s] = 1; }
      }
    }
    for (uint32_t s : nxt) in_next[s] = 0;
    cur.swap(nxt);
  }
  return rounds;
}

uint64_t oracle_mer_merge(const uint32_t* wl, uint64_t n, const uint32_t* dst, uint64_t nd,
                          uint32_t* next, uint64_t cap, uint64_t* head_n) {
  uint64_t head = (n <= 32) ? n : (n / 32) * 32;     // Alg. 3 l.8; Fig. 7: 36 -> 32 (A13)
  if (head_n) *head_n = head;
  std::vector<uint32_t> tail(wl + head, wl + n), out;
  for (uint64_t i = 0; i < nd; ++i) {
    uint32_t x = dst[i];
    if (std::find(tail.begin(), tail.end(), x) != tail.end()) continue;  // already in the tail
    if (std::find(out.begin(), out.end(), x) != out.end()) continue;    // repetition
    out.push_back(x);
  }
  for (uint32_t x : tail)
    if (std::find(out.begin(), out.end(), x) == out.end()) out.push_back(x);
  for (uint64_t i = 0; i < out.size() && i < cap; ++i) next[i] = out[i];
  return out.size();
}

}  // extern "C"
