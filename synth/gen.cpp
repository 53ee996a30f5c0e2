// gen.cpp — seeded synthetic Android-app-shaped ICFG generator (input construction only).
//
// Shared by the oracle and the CUDA path through synth/generator.py; holds none of the
// method's arithmetic (no transfer function, no union, no fixed point).  Shapes follow
// components with an environment method each (Eq. 1,
// PAPER.md:351-355), modules of consecutive methods with pre-determined instance/slot pools
// (PAPER.md:859-867), structured method bodies (sequences, if/else diamonds, switches,
// while loops), call sites with CALL/RETSITE/C2R/RET edges, virtual fan-out, recursion
// cycles and deep call chains.  The statement mix is a performance knob (the paper is silent).
#include <algorithm>
#include <cmath>
#include <cstdint>
#include <cstring>
#include <unordered_set>
#include <vector>

extern "C" {
typedef struct {
  uint64_t seed;
  uint32_t n_methods;          // total methods
  uint32_t stmts_per_method;   // mean statements per method (nodes ~ 1.5x)
  uint32_t n_components;       // K independent components (entries)
  uint32_t methods_per_module;
  uint32_t q_cap;              // instance pool size per module (<= 512)
  uint32_t n_types;            // reference types (plus array / const types)
  uint32_t n_fields;           // field ids (0 = ARR)
  uint32_t fields_per_type;    // max fields per reference type
  uint32_t statics_per_module; // own statics per module
  uint32_t temps_per_method;   // temporaries per method
  uint32_t call_span;          // forward window of callees (controls call depth)
  double p_recursion;          // probability a call targets an earlier method (cycles)
  double mix[13];              // PRIM COPY CONST NEW FLOAD FSTORE ALOAD ASTORE SLOAD SSTORE CALL NOP (12) + p_branch
} gen_params;
}

namespace {

enum { NOP, ENTRY, EXIT, RETSITE, CALL, PRIM, CONST, NEW, COPY, SLOAD, SSTORE, RETV, FLOAD, FSTORE, ALOAD, ASTORE };
enum { E_INTRA, E_CALL, E_RET, E_C2R };

struct Rng {
  uint64_t s;
  uint64_t next() {
    uint64_t z = (s += 0x9e3779b97f4a7c15ULL);
    z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ULL;
    z = (z ^ (z >> 27)) * 0x94d049bb133111ebULL;
    return z ^ (z >> 31);
  }
  double uni() { return (next() >> 11) * (1.0 / 9007199254740992.0); }
  uint32_t below(uint32_t n) { return n ? (uint32_t)((next() >> 32) * (uint64_t)n >> 32) : 0; }
};

struct Region { int first, last; };

struct Gen {
  gen_params P;
  Rng R;
  // output
  std::vector<uint8_t> node_kind;
  std::vector<uint32_t> node_method;
  std::vector<int32_t> node_ops;
  std::vector<std::vector<std::pair<uint32_t, uint8_t>>> succ;
  std::vector<std::vector<int32_t>> call_args;
  std::vector<uint32_t> m_entry, m_exit, m_module, m_nlocals, m_nparams;
  std::vector<std::vector<uint32_t>> mod_insts, mod_statics;
  std::vector<int32_t> inst_type;
  std::vector<std::vector<uint32_t>> type_fields;
  std::vector<uint32_t> entries;
  // generation state
  std::vector<uint64_t> local_base;
  uint64_t L_total = 0;
  uint32_t n_statics = 0;
  std::vector<uint32_t> ref_types, arr_types, const_types;
  std::vector<std::vector<uint32_t>> mod_types;        // hot types per module
  std::vector<std::vector<uint32_t>> mod_sites;        // instances created by each module
  std::vector<std::unordered_set<uint32_t>> mod_neighbors;
  std::vector<std::vector<uint32_t>> planned;          // planned callees per method
  std::vector<std::vector<uint32_t>> by_arity[9];      // per component: methods by arity (0..8)
  std::vector<uint32_t> comp_of_method, comp_begin, comp_end;
  std::vector<std::pair<uint32_t, uint32_t>> pending_ret;  // (callee, retsite) RET edges
  std::vector<std::pair<uint32_t, uint32_t>> pending_call; // (call node, callee) CALL edges
  // per-method scratch
  uint32_t cm = 0, cmod = 0, cur_nl = 0, cur_np = 0;
  std::vector<uint32_t> defined;

  int node(uint32_t m, uint8_t kind, int32_t a = -1, int32_t b = -1, int32_t c = -1, int32_t d = -1) {
    node_kind.push_back(kind);
    node_method.push_back(m);
    node_ops.push_back(a); node_ops.push_back(b); node_ops.push_back(c); node_ops.push_back(d);
    succ.emplace_back();
    call_args.emplace_back();
    return (int)node_kind.size() - 1;
  }
  void edge(int a, int b, uint8_t k = E_INTRA) { succ[a].push_back({(uint32_t)b, k}); }

  int32_t loc(uint32_t i) { return (int32_t)(local_base[cm] + i); }
  uint32_t any_local() { return R.below(cur_nl - 1); }            // never RET
  uint32_t use_local() {
    if (!defined.empty() && R.uni() < 0.75) return defined[R.below((uint32_t)defined.size())];
    return any_local();
  }
  uint32_t def_local() {
    uint32_t lo = cur_np, n = cur_nl - 1 - cur_np;                 // temporaries
    uint32_t v = n ? lo + R.below(n) : any_local();
    defined.push_back(v);
    if (defined.size() > 12) defined.erase(defined.begin());
    return v;
  }
  uint32_t pick_field() {
    const auto& ts = mod_types[cmod];
    const auto& fl = type_fields[ts[R.below((uint32_t)ts.size())]];
    return fl.empty() ? 1 : fl[R.below((uint32_t)fl.size())];
  }
  int32_t static_gid() {
    const auto& s = mod_statics[cmod];
    return s.empty() ? -1 : (int32_t)(L_total + s[R.below((uint32_t)s.size())]);
  }
  uint32_t new_instance(bool is_const) {
    uint32_t t;
    if (is_const) t = const_types[R.below((uint32_t)const_types.size())];
    else if (R.uni() < 0.08) t = arr_types[R.below((uint32_t)arr_types.size())];
    else t = mod_types[cmod][R.below((uint32_t)mod_types[cmod].size())];
    inst_type.push_back((int32_t)t);
    uint32_t o = (uint32_t)inst_type.size() - 1;
    mod_sites[cmod].push_back(o);
    return o;
  }

  Region call_stmt(uint32_t first_target) {
    // targets: the planned/first target plus virtual fan-out with the same arity (C3)
    const uint32_t ar = m_nparams[first_target];
    std::vector<uint32_t> targets{first_target};
    double u = R.uni();
    uint32_t fan = u < 0.80 ? 1 : (u < 0.98 ? 2 + R.below(3) : 5 + R.below(12));
    const auto& cands = by_arity[ar][comp_of_method[cm]];
    for (uint32_t tries = 0; targets.size() < fan && tries < 4 * fan && cands.size() > 1; ++tries) {
      uint32_t t = cands[R.below((uint32_t)cands.size())];
      if (t == comp_begin[comp_of_method[cm]]) continue;
      if (t > cm + P.call_span * 4 || (t < cm && R.uni() > P.p_recursion * 4)) continue;
      if (std::find(targets.begin(), targets.end(), t) == targets.end()) targets.push_back(t);
    }
    int32_t lhs = R.uni() < 0.7 ? loc(def_local()) : -1;
    int c = node(cm, CALL, lhs);
    int r = node(cm, RETSITE, lhs, -1, -1, c);
    // actuals: a used local (85 %) or a non-reference value (-1); 15 % of the calls with two or
    // more parameters pass one local for several of them (setPadding(p, p, p, p)-style), so a
    // source row can feed many parameter rows (C3)
    if (ar >= 2 && R.uni() < 0.15) {
      const int32_t rep = loc(use_local());
      for (uint32_t j = 0; j < ar; ++j) call_args[c].push_back(R.uni() < 0.8 ? rep : (R.uni() < 0.5 ? -1 : loc(use_local())));
    } else {
      for (uint32_t j = 0; j < ar; ++j)
        call_args[c].push_back(R.uni() < 0.85 ? loc(use_local()) : -1);
    }
    for (uint32_t t : targets) {
      pending_call.push_back({(uint32_t)c, t});               // m_entry[t] may not exist yet
      pending_ret.push_back({t, (uint32_t)r});
      mod_neighbors[cmod].insert(m_module[t]);
      mod_neighbors[m_module[t]].insert(cmod);
    }
    edge(c, r, E_C2R);
    return {c, r};
  }

  uint32_t random_target() {
    const uint32_t k = comp_of_method[cm];
    const uint32_t b = comp_begin[k], e = comp_end[k];
    if (R.uni() < P.p_recursion && cm > b + 1) {             // cycle of length 1..5
      uint32_t back = 1 + R.below(std::min<uint32_t>(5, cm - b - 1));
      return cm - back + 1;                                   // > b: never the environment method
    }
    uint32_t lo = cm + 1, hi = std::min<uint64_t>(e, (uint64_t)cm + 1 + P.call_span);
    if (lo >= hi) return (cm > b + 1) ? b + 1 + R.below(cm - b - 1) : cm;
    return lo + R.below(hi - lo);
  }

  Region stmt() {
    const double* w = P.mix;
    double tot = 0;
    for (int i = 0; i < 12; ++i) tot += w[i];
    double u = R.uni() * tot;
    int pick = 0;
    while (pick < 11 && u >= w[pick]) { u -= w[pick]; ++pick; }
    int n;
    switch (pick) {
      case 0: n = node(cm, PRIM, loc(def_local())); break;
      case 1: { uint32_t w2 = use_local(); n = node(cm, COPY, loc(def_local()), loc(w2)); break; }
      case 2: {
        bool null = R.uni() < 0.35;
        uint32_t o = null ? 0 : new_instance(true);
        n = node(cm, CONST, loc(def_local()), -1, -1, (int32_t)o);
        break;
      }
      case 3: { uint32_t o = new_instance(false); n = node(cm, NEW, loc(def_local()), -1, -1, (int32_t)o); break; }
      case 4: { uint32_t w2 = use_local(); n = node(cm, FLOAD, loc(def_local()), loc(w2), (int32_t)pick_field()); break; }
      case 5: { uint32_t v = use_local(), w2 = use_local(); n = node(cm, FSTORE, loc(v), loc(w2), (int32_t)pick_field()); break; }
      case 6: { uint32_t w2 = use_local(); n = node(cm, ALOAD, loc(def_local()), loc(w2), 0); break; }
      case 7: { uint32_t v = use_local(), w2 = use_local(); n = node(cm, ASTORE, loc(v), loc(w2), 0); break; }
      case 8: {
        int32_t g = static_gid();
        n = g < 0 ? node(cm, PRIM, loc(def_local())) : node(cm, SLOAD, loc(def_local()), g);
        break;
      }
      case 9: {
        int32_t g = static_gid();
        n = g < 0 ? node(cm, NOP) : node(cm, SSTORE, g, loc(use_local()));
        break;
      }
      case 10: {
        uint32_t t;
        if (!planned[cm].empty()) { t = planned[cm].back(); planned[cm].pop_back(); }
        else t = random_target();
        if (t == comp_begin[comp_of_method[cm]]) { n = node(cm, NOP); break; }
        return call_stmt(t);
      }
      default: n = node(cm, NOP); break;
    }
    return {n, n};
  }

  // structured body: sequences, if/else and switch diamonds, while loops (nesting <= 3)
  Region seq(int budget, int depth) {
    Region out{-1, -1};
    while (budget > 0) {
      Region r;
      int used = 1;
      double u = R.uni();
      const double pb = P.mix[12];
      if (depth < 3 && budget >= 4 && u < pb) {                 // if / switch
        int k = R.uni() < 0.85 ? 2 : 3 + (int)R.below(3);
        int cond = node(cm, NOP), join = node(cm, NOP);
        int part = std::max(1, (budget - 2) / (k + 1));
        for (int b = 0; b < k; ++b) {
          if (b == k - 1 && k == 2 && R.uni() < 0.3) { edge(cond, join); continue; }   // if without else
          Region br = seq(1 + (int)R.below(part), depth + 1);
          edge(cond, br.first); edge(br.last, join);
          used += part;
        }
        r = {cond, join};
        used += 2;
      } else if (depth < 3 && budget >= 3 && u < pb * 1.6) {      // while loop
        int head = node(cm, NOP);
        Region body = seq(1 + (int)R.below(std::max(1, budget / 2)), depth + 1);
        edge(head, body.first); edge(body.last, head);
        r = {head, head};
        used += 1 + budget / 3;
      } else {
        r = stmt();
      }
      if (out.first < 0) out.first = r.first; else edge(out.last, r.first);
      out.last = r.last;
      budget -= used;
    }
    if (out.first < 0) { int n = node(cm, NOP); out = {n, n}; }
    return out;
  }

  void run() {
    R.s = P.seed * 0x2545F4914F6CDD1DULL + 0x1234567ULL;
    const uint32_t M = std::max<uint32_t>(P.n_methods, 1), K = std::max<uint32_t>(1, std::min(P.n_components, M));
    // types: ref types with fields, array types (ARR), const types (String/Class: no fields)
    inst_type.push_back(-1);                                   // NULL
    const uint32_t NF = std::max<uint32_t>(P.n_fields, 2);
    for (uint32_t t = 0; t < std::max<uint32_t>(P.n_types, 1); ++t) {
      uint32_t nf = 1 + R.below(std::max<uint32_t>(P.fields_per_type, 1));
      std::vector<uint32_t> f;
      while (f.size() < nf) {
        uint32_t x = 1 + R.below(NF - 1);
        if (std::find(f.begin(), f.end(), x) == f.end()) f.push_back(x);
      }
      std::sort(f.begin(), f.end());
      ref_types.push_back((uint32_t)type_fields.size());
      type_fields.push_back(f);
    }
    for (int i = 0; i < 2; ++i) { arr_types.push_back((uint32_t)type_fields.size()); type_fields.push_back({0}); }
    for (int i = 0; i < 2; ++i) { const_types.push_back((uint32_t)type_fields.size()); type_fields.push_back({}); }
    // components, modules, methods
    comp_begin.resize(K); comp_end.resize(K);
    for (uint32_t k = 0; k < K; ++k) { comp_begin[k] = (uint32_t)((uint64_t)M * k / K); comp_end[k] = (uint32_t)((uint64_t)M * (k + 1) / K); }
    comp_of_method.resize(M);
    uint32_t n_mod = 0;
    for (uint32_t k = 0; k < K; ++k) {
      for (uint32_t m = comp_begin[k]; m < comp_end[k]; ++m) {
        comp_of_method[m] = k;
        if ((m - comp_begin[k]) % std::max<uint32_t>(P.methods_per_module, 1) == 0) ++n_mod;
        m_module.push_back(n_mod - 1);
      }
    }
    mod_types.resize(n_mod); mod_sites.resize(n_mod); mod_neighbors.resize(n_mod); mod_statics.resize(n_mod);
    for (uint32_t d = 0; d < n_mod; ++d) {
      uint32_t nt = 2 + R.below(3);
      for (uint32_t i = 0; i < nt; ++i) mod_types[d].push_back(ref_types[R.below((uint32_t)ref_types.size())]);
      for (uint32_t i = 0; i < P.statics_per_module; ++i) mod_statics[d].push_back(n_statics++);
    }
    // statics are also shared with the next module of the same component (cross-module flow)
    for (uint32_t d = 0; d + 1 < n_mod; ++d)
      if (!mod_statics[d].empty() && R.uni() < 0.5) mod_statics[d + 1].push_back(mod_statics[d][0]);
    for (auto& s : mod_statics) { std::sort(s.begin(), s.end()); s.erase(std::unique(s.begin(), s.end()), s.end()); }
    m_nparams.resize(M); m_nlocals.resize(M);
    for (int a = 0; a < 9; ++a) by_arity[a].resize(K);
    for (uint32_t m = 0; m < M; ++m) {
      double u = R.uni();
      // arity 0..8 (Android APIs take up to ~8 arguments; 8 % of the methods take 4 or more)
      uint32_t np = m == comp_begin[comp_of_method[m]] ? 0
                  : (u < 0.2 ? 0 : u < 0.53 ? 1 : u < 0.80 ? 2 : u < 0.92 ? 3 : 4 + R.below(5));
      m_nparams[m] = np;
      m_nlocals[m] = np + std::max<uint32_t>(P.temps_per_method, 1) + 1;
      by_arity[np][comp_of_method[m]].push_back(m);
    }
    local_base.assign(M + 1, 0);
    for (uint32_t m = 0; m < M; ++m) local_base[m + 1] = local_base[m] + m_nlocals[m];
    L_total = local_base[M];
    // planned spine calls: every non-environment method gets a caller inside its component
    planned.resize(M);
    for (uint32_t k = 0; k < K; ++k)
      for (uint32_t j = comp_begin[k] + 1; j < comp_end[k]; ++j) {
        uint32_t lo = j > comp_begin[k] + P.call_span ? j - P.call_span : comp_begin[k];
        planned[lo + R.below(j - lo)].push_back(j);
      }
    // entry/exit nodes are created first per method, then its body
    m_entry.resize(M); m_exit.resize(M);
    for (uint32_t m = 0; m < M; ++m) {
      cm = m; cmod = m_module[m]; cur_nl = m_nlocals[m]; cur_np = m_nparams[m];
      defined.clear();
      for (uint32_t i = 0; i < cur_np; ++i) defined.push_back(i);
      m_entry[m] = (uint32_t)node(m, ENTRY);
      m_exit[m] = (uint32_t)node(m, EXIT);
      int budget = (int)(P.stmts_per_method / 2 + R.below(P.stmts_per_method + 1));
      budget = std::max<int>(budget, (int)planned[m].size() * 2 + 1);
      Region body = seq(budget, 0);
      while (!planned[m].empty()) {                             // remaining spine calls
        Region c = call_stmt(planned[m].back());
        planned[m].pop_back();
        edge(body.last, c.first);
        body.last = c.last;
      }
      edge((int)m_entry[m], body.first);
      int last = body.last;
      if (R.uni() < 0.7) {                                      // returns a reference
        int rv = node(m, RETV, -1, loc(use_local()));
        edge(last, rv);
        last = rv;
      }
      edge(last, (int)m_exit[m]);
    }
    for (auto& pc : pending_call) edge((int)pc.first, (int)m_entry[pc.second], E_CALL);
    for (auto& pr : pending_ret) edge((int)m_exit[pr.first], (int)pr.second, E_RET);
    // pools: own sites + NULL + instances of neighbour modules, up to q_cap
    mod_insts.resize(n_mod);
    for (uint32_t d = 0; d < n_mod; ++d) {
      std::vector<uint32_t> pool{0};
      pool.insert(pool.end(), mod_sites[d].begin(), mod_sites[d].end());
      std::vector<uint32_t> cand;
      for (uint32_t nb : mod_neighbors[d]) if (nb != d) cand.insert(cand.end(), mod_sites[nb].begin(), mod_sites[nb].end());
      for (uint32_t i = 0; i < cand.size(); ++i) std::swap(cand[i], cand[i + R.below((uint32_t)(cand.size() - i))]);
      for (uint32_t o : cand) { if (pool.size() >= P.q_cap) break; pool.push_back(o); }
      std::sort(pool.begin(), pool.end());
      pool.erase(std::unique(pool.begin(), pool.end()), pool.end());
      mod_insts[d] = pool;
    }
    for (uint32_t k = 0; k < K; ++k) entries.push_back(m_entry[comp_begin[k]]);
  }
};

}  // namespace

struct gen_result {
  Gen g;
  std::vector<uint64_t> row_ptr, call_arg_ptr, module_inst_ptr, module_static_ptr, type_field_ptr;
  std::vector<uint32_t> col, module_insts, module_statics, type_fields;
  std::vector<uint8_t> edge_kind;
  std::vector<int32_t> call_args;
  uint64_t scalars[4];   // n_statics, n_fields, own-site overflow count, n_modules
};

extern "C" {

// Generate one app; returns NULL only on allocation failure.
gen_result* gen_app(const gen_params* p) {
  gen_result* r = new gen_result;
  Gen& g = r->g;
  g.P = *p;
  if (g.P.q_cap < 2) g.P.q_cap = 2;
  if (g.P.q_cap > 512) g.P.q_cap = 512;
  g.run();
  // pools must hold every own site (V1): sites beyond q_cap turn into PRIM statements
  uint64_t overflow = 0;
  for (uint32_t d = 0; d < g.mod_insts.size(); ++d) {
    if (g.mod_insts[d].size() <= g.P.q_cap) continue;
    g.mod_insts[d].resize(g.P.q_cap);
  }
  for (size_t n = 0; n < g.node_kind.size(); ++n) {
    uint8_t k = g.node_kind[n];
    if ((k == NEW || k == CONST) && g.node_ops[4 * n + 3] != 0) {
      uint32_t d = g.m_module[g.node_method[n]];
      const auto& pool = g.mod_insts[d];
      if (!std::binary_search(pool.begin(), pool.end(), (uint32_t)g.node_ops[4 * n + 3])) {
        g.node_kind[n] = PRIM;
        g.node_ops[4 * n + 3] = -1;
        ++overflow;
      }
    }
  }
  const size_t N = g.node_kind.size();
  r->row_ptr.assign(N + 1, 0);
  r->call_arg_ptr.assign(N + 1, 0);
  for (size_t n = 0; n < N; ++n) {
    for (auto& e : g.succ[n]) { r->col.push_back(e.first); r->edge_kind.push_back(e.second); }
    r->row_ptr[n + 1] = r->col.size();
    for (int32_t a : g.call_args[n]) r->call_args.push_back(a);
    r->call_arg_ptr[n + 1] = r->call_args.size();
  }
  r->module_inst_ptr.push_back(0);
  for (auto& v : g.mod_insts) { r->module_insts.insert(r->module_insts.end(), v.begin(), v.end()); r->module_inst_ptr.push_back(r->module_insts.size()); }
  r->module_static_ptr.push_back(0);
  for (auto& v : g.mod_statics) { r->module_statics.insert(r->module_statics.end(), v.begin(), v.end()); r->module_static_ptr.push_back(r->module_statics.size()); }
  r->type_field_ptr.push_back(0);
  for (auto& v : g.type_fields) { r->type_fields.insert(r->type_fields.end(), v.begin(), v.end()); r->type_field_ptr.push_back(r->type_fields.size()); }
  r->scalars[0] = g.n_statics;
  r->scalars[1] = std::max<uint32_t>(g.P.n_fields, 2);
  r->scalars[2] = overflow;
  r->scalars[3] = g.mod_insts.size();
  return r;
}

// Array views in synth/icfg.py ARRAY_FIELDS order; lens in elements.
void gen_arrays(gen_result* r, const void** ptrs, uint64_t* lens, uint64_t* scalars) {
  Gen& g = r->g;
#define V(i, vec) ptrs[i] = (vec).data(); lens[i] = (vec).size();
  V(0, r->row_ptr) V(1, r->col) V(2, r->edge_kind) V(3, g.node_kind) V(4, g.node_method) V(5, g.node_ops)
  V(6, r->call_arg_ptr) V(7, r->call_args) V(8, g.m_entry) V(9, g.m_exit) V(10, g.m_module)
  V(11, g.m_nlocals) V(12, g.m_nparams) V(13, r->module_inst_ptr) V(14, r->module_insts)
  V(15, r->module_static_ptr) V(16, r->module_statics) V(17, g.inst_type) V(18, r->type_field_ptr)
  V(19, r->type_fields) V(20, g.entries)
#undef V
  for (int i = 0; i < 4; ++i) scalars[i] = r->scalars[i];
}

void gen_free(gen_result* r) { delete r; }

}  // extern "C"
