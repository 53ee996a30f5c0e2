// internal.cuh — device layout shared by the loader (loader.cu) and the kernels (kernels.cu).
// Not part of the C ABI.  DESIGN.md §4 describes this layout.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

#include "../../include/gdroid.h"

namespace gd {

constexpr int MAXW = 8;            // max 64-bit words per fact row: |Q_m| <= 512 instances
constexpr int NCLS = 5;            // GRP classes + 2 interprocedural classes
enum Cls : uint8_t { C_ONETIME = 0, C_SINGLE = 1, C_DOUBLE = 2, C_CALL = 3, C_EXIT = 4 };
constexpr int CNT_STRIDE = 8;      // counts[rot * CNT_STRIDE + cls]; slot CNT_NODES = nodes queued
constexpr int CNT_NODES = 5;
// D.bar words: [0] arrivals and [1] generation of the grid barrier, [3] hybrid hand-over round,
// [4..6] SBDA claim cursors; the worklist-empty flag that every warp reads after the barrier
// sits in its own 128-byte line, away from the barrier's atomics and pollers.
constexpr int BAR_DONE = 32;
#ifndef GD_HIOCC_NODES
#define GD_HIOCC_NODES (1u << 17)
#endif
constexpr uint32_t HIOCC_NODES = GD_HIOCC_NODES;   // batches this large are item-throughput bound
#ifndef GD_THREADS
#define GD_THREADS 256
#endif
constexpr int THREADS = GD_THREADS; // fixed-point kernel block size
#ifndef GD_NMASK
#define GD_NMASK 0             // narrow blocks: word-occupancy masks in D.smask (2 words per node
                               // cover words 0..127); readers load only non-zero words of IN(src).
                               // Correct (all GPU tests pass) but +6 % on corpus200, +4 % on median
                               // (profiles/r02_ab_nmask.log): off, D.smask not allocated
#endif
constexpr uint32_t NMW = 2;    // mask words per node
constexpr int WARPS = THREADS / 32;

// One ICFG node (64 B).  Row indices r* are relative to the node's fact block (method-local
// rows first, then the module's global rows), resolved by the loader, and the block's layout
// is copied in so a visit needs no method/module lookups.
struct __align__(16) NodeRec {
  uint64_t off;      // word offset of IN(n) in the fact store
  uint32_t e0, e1;   // out-edge range [e0, e1) in the edge array
  uint8_t kind;      // gdroid_node_kind
  uint8_t cls;       // Cls
  uint8_t logW;      // log2 words per row
  uint8_t n_inl;     // edges of chunk 0 held inline in InlEdge[4 * n ..] (all INTRA/C2R, narrow
                     // block of <= 128 words), 0 = read them from the edge array
  int32_t r0;        // lhs row (PRIM/CONST/NEW/COPY/SLOAD/RETV/FLOAD/ALOAD), static row (SSTORE),
                     // base row (FSTORE/ASTORE), lhs row of the call (CALL/RETSITE) or -1
  int32_t r1;        // rhs row (COPY/SLOAD/SSTORE/RETV), w row (FLOAD/ALOAD/FSTORE/ASTORE),
                     // n_params of the method (ENTRY), argument rows r1..r3 (CALL with <= 3 args)
  int32_t r2;        // field id (FLOAD/FSTORE; F_ARR for ALOAD/ASTORE)
  int32_t r3;        // instance column (CONST/NEW); field-row table offset (FLOAD/FSTORE/ALOAD/ASTORE)
  uint32_t B;        // words of the block = (L + n_glob) << logW
  uint32_t L;        // method-local rows (params, temps, RET)
  uint32_t n_stat;   // module static rows
  uint32_t col_off;  // module column tables
  uint32_t grow_off; // module global-row tables
  uint16_t n_cols;   // |Q| of the module
  uint16_t app;      // index of the app inside a batch
  uint32_t local_base; // app-local slot gid of the method's local 0 (digest / readback)
};
static_assert(sizeof(NodeRec) == 64, "NodeRec must be 64 bytes");

// Wide blocks (modules with more than 64 instances, logW >= 1) carry a row-occupancy bitmap
// after the rows: bit r set = row r may be non-zero.  Writers set it, readers visit only the
// flagged rows (a fact written after the reader's bitmap load is re-processed next round,
// because its writer also queued the node).
__host__ __device__ __forceinline__ uint32_t occ_offset(uint32_t B) { return (B + 3u) & ~3u; }
__host__ __device__ __forceinline__ uint32_t occ_words(uint32_t rows) { return (rows + 63u) >> 6; }

// Work items.  A node's out-edges are split into chunks of ebs(deg) edges (at most 32 chunks
// per node); a queue entry is (node << 5) | chunk.  High-degree nodes (method exits with many
// return sites, virtual calls with many targets) thus spread over several warps.
// INTRA/C2R edges share one transfer evaluation, so their chunks hold up to 4 edges; CALL
// and RET edges each re-map the whole block, so CALL and EXIT nodes get one edge per chunk.
constexpr uint32_t EDGES_PER_CHUNK = 4;
// Wide blocks (logW >= 1) are never split: their visit consumes Δ(src) once (semi-naive, DESIGN.md
// §5.5), so one warp must propagate it along every out-edge.
__host__ __device__ __forceinline__ uint32_t chunk_edges(uint32_t deg, uint32_t cls, uint32_t logW) {
  if (logW >= 1) return deg > 0 ? deg : 1u;
  const uint32_t e = (deg + 31) >> 5;
  const uint32_t lo = (cls == 3u || cls == 4u) ? 1u : EDGES_PER_CHUNK;   // C_CALL, C_EXIT
  return e > lo ? e : lo;
}
__host__ __device__ __forceinline__ uint32_t n_chunks_of(uint32_t deg, uint32_t cls, uint32_t logW) {
  return deg == 0 ? 1u : (deg + chunk_edges(deg, cls, logW) - 1) / chunk_edges(deg, cls, logW);
}

// Chunk 0's INTRA/C2R out-edges of a narrow node, held beside its NodeRec (4 x 16 B = one
// 64-byte record per node, loaded in the same memory hop as the NodeRec): an intra-method edge
// keeps the source's block layout, so only the destination id, info and fact offset are needed.
struct __align__(16) InlEdge {
  uint32_t dst;
  uint32_t info;       // as Edge::info
  uint64_t off;        // fact-block word offset of dst
};
static_assert(sizeof(InlEdge) == 16, "InlEdge must be 16 bytes");
constexpr uint32_t INL_MAX_B = 128;   // inline path: narrow source blocks of at most 128 words

// Per-app table bases of a batch: the loader stages each app's node tables with app-local
// indices, k_rebase adds these.
struct __align__(16) AppBase {
  uint64_t fact;
  uint32_t edge, meth, mod, col, grow, frow, args, pad;
};

struct __align__(16) MethRec {
  uint32_t n_locals, n_params, module, local_base;   // local_base: app-local slot gid of local 0
};

struct __align__(16) ModRec {
  uint32_t n_cols;     // |Q| (column 0 is NULL)
  uint32_t W, logW;    // 64-bit words per row (power of two) and log2
  uint32_t n_stat;     // static rows (global rows [0, n_stat))
  uint32_t n_glob;     // n_stat + heap rows
  uint32_t col_off;    // into col_gid / col_type / col_hbase
  uint32_t grow_off;   // into grow_gid / grow_col / grow_field
  uint32_t pad;
};

// One out-edge (32 B) with the destination's layout copied in, so a CALL/RET edge needs no
// lookup of the destination node.
struct __align__(16) Edge {
  uint32_t dst;
  uint32_t info;       // kind (2 bits) | class of dst << 2 (3 bits) | (chunks of dst - 1) << 5
                       // | INFO_WIDE (dst block is wide)
  uint64_t off;        // fact-block word offset of dst
  uint32_t B;          // dst block words
  uint16_t L;          // dst method-local rows
  uint8_t logW;        // dst log2 words per row
  uint8_t pad;
  int32_t aux;         // CALL: n_params of the callee; RET: lhs(c) row at the return site (-1)
  uint32_t xoff;       // projection π: xmap offset (colmap |Q_src| then rowmap n_glob(dst)),
                       // 0xffffffff = same module (identity)
};
static_assert(sizeof(Edge) == 32, "Edge must be 32 bytes");
constexpr uint32_t INFO_WIDE = 1u << 10;
constexpr uint32_t NO_XMAP = 0xffffffffu;

// Scheduling switches (gdroid_build_opts.variant).  GRP off = one worklist
// segment in arrival order; MER = head/tail split with the tail merged into the next worklist
// (Fig. 7); CONT = depth-first continuation into wide successors.
constexpr uint32_t F_GRP = 1u, F_MER = 2u, F_CONT = 4u;

struct DevStats {
  unsigned long long rounds, visits, alg_bytes, dense_bytes, atomics, hist[3], limit_hit, seed_err;
  unsigned long long phase[8];  // GD_PHASES builds: cycles in setup / edges / push / round end, items
};

struct Dev {
  const NodeRec* nodes;
  const MethRec* meths;
  const ModRec* mods;
  const uint32_t* row_ptr;
  const Edge* edges;
  const InlEdge* inl;           // [4 N] chunk-0 INTRA/C2R edges (NodeRec::n_inl of them valid)
  const uint32_t* arg_ptr;
  const int32_t* args;
  const uint32_t* col_gid;
  const int32_t* col_type;
  const uint32_t* col_hbase;
  const uint32_t* grow_gid;
  const int32_t* grow_col;
  const int32_t* grow_field;
  const uint32_t* tf_ptr;
  const uint32_t* tf;
  const int32_t* xmap;          // projection tables (see Edge::xoff)
  const uint32_t* app_node_base;
  const uint32_t* entries;      // global node ids of all component entries of all apps
  const uint32_t* node_method;  // [N] (digest / readback only)
  const int32_t* frow;          // field-row tables: frow[r3 + c] = global row of (col c, f) | -1
  uint64_t* facts;
  uint64_t* delta;              // wide batches: Δ store, same layout as facts (bits that reached
                                // IN(n) since n's last visit); nullptr if narrow
  uint64_t* smask;              // [NMW N] narrow word-occupancy masks (GD_NMASK): bit w = word w may be non-zero
  uint32_t* stamp;              // [N] last round a node was queued for (0 = never)
  uint32_t* cont;               // [N] last round a warp continued into the node (0 = never)
  uint32_t* queue;              // [3][n_chunks] rotating class-segmented worklists of
                                // (node << 5 | chunk) entries
  uint32_t* counts;             // [3][CNT_STRIDE]
  DevStats* stats;
  uint32_t* bar;                // grid barrier {count, generation}
  uint64_t* node_digest;        // [N]
  uint32_t* node_popc;          // [N] facts per node, written by k_digest (readback sizes)
  unsigned long long* app_digest; // [n_apps]
  uint64_t n_words;             // fact store size in words
  uint32_t n_nodes;
  uint32_t n_chunks;
  uint32_t n_entries;
  uint32_t seg[NCLS + 1];       // class segment starts inside one queue
  uint32_t max_rounds;
  uint32_t wide;                // max log2(words per row) over the batch's modules: 0 = all narrow,
                                // >= 1: some module has > 64 instances (row-occupancy path)
  uint32_t hiocc;               // 1: launch the 4-CTA/SM narrow instantiation (batches >= HIOCC_NODES)
  const uint32_t* seed_nodes;   // staged seed nodes queued by k_seed (incremental builds)
  const uint32_t* seed_pairs;   // [3 n] (node, slot gid, instance gid) OR-ed in by k_apply_seeds
  uint32_t n_seed_nodes, n_seed_pairs;
  uint32_t push_entries;        // 1: k_seed queues the component entries (fresh builds)
  uint32_t round0;              // first round of this build / launch (1 for a fresh build)
  // SBDA schedule (variant GDROID_V_SBDA), set up at its first build:
  const uint32_t* meth_node_ptr;  // [n_meths+1] CSR of each method's nodes
  const uint32_t* meth_nodes;
  uint32_t* claim;              // [n_meths] last pass a CTA claimed the method
  unsigned long long* lstamp;   // [N] last local round a node was queued in (pass << 32 | counter)
  uint32_t n_meths;
  uint32_t hyb;                 // 1: hybrid launch sequence: start at round bar[3], return if it is 0
  uint32_t sw_lo, sw_hi;        // hybrid: leave at the start of a round with < sw_lo / >= sw_hi items
                                // (bar[3] = that round), 0 = off
  uint32_t flags;               // F_* scheduling switches of the build (ablation variants)
  uint32_t count;               // 1: evaluate the byte models (alg/dense bytes, atomics) on the device
  unsigned long long* trace;    // optional per-round trace: {globaltimer ns, items << 32 | nodes}
  uint32_t trace_cap;           // rounds recorded (0 = off)
};

// ---- PLAIN variant (plain.cu): set-based facts, thread per node (Alg. 2)
struct __align__(16) SetDesc {
  uint64_t off;      // word offset of the node's sorted pair array in the heap
  uint32_t size;     // pairs stored
  uint32_t cap;      // pairs allocated
};
static_assert(sizeof(SetDesc) == 16, "SetDesc must be 16 bytes");

struct PlainDev {
  // input: device copies of one app's gdroid_icfg_desc arrays (+ two host-computed prefixes)
  const uint64_t* row_ptr; const uint32_t* col; const uint8_t* ekind; const uint8_t* nkind;
  const uint32_t* nmeth; const int32_t* ops; const uint64_t* arg_ptr; const int32_t* args;
  const uint64_t* local_base;   // [M+1] prefix of method_n_locals
  const uint32_t* n_params; const uint32_t* mmod;
  const uint64_t* inst_ptr; const uint32_t* insts; const uint64_t* stat_ptr; const uint32_t* statics;
  const int32_t* inst_type; const uint64_t* tf_ptr; const uint32_t* tfields;
  const uint64_t* heap_base;    // [I+1] prefix of |F(t(o))|
  const uint32_t* entries;
  uint64_t L_total, G;
  uint32_t n_nodes, n_instances, n_entries, max_rounds;
  // state
  SetDesc* sets; uint32_t* locks; uint64_t* heap; unsigned long long* heap_top; uint64_t heap_cap;
  uint64_t* scratch; uint64_t maxset;   // per thread: 3 buffers of maxset pairs
  uint32_t* stamp; uint32_t* queue; uint32_t* counts; uint32_t* bar; uint32_t* err;
  DevStats* stats;
  uint64_t* node_digest; unsigned long long* app_digest;
  // CELL variant: the paper's cell-major per-method matrix (Fig. 5b,
  // PAPER.md:871-904): method m owns rows (locals, then the module's global rows in gid order)
  // x columns (its module's instance pool); cell (r, c) is an n_m-bit mask over m's nodes.
  uint32_t cell;                // 1: this build runs on the cell store instead of the pair sets
  uint32_t n_methods;
  uint64_t* cells;              // the cell store (cell_words words)
  uint64_t cell_words;
  const uint64_t* m_coff;       // [M] word offset of method m's matrix
  const uint32_t* m_rows;       // [M] |P_m|
  const uint32_t* m_cols;       // [M] |Q_m|
  const uint32_t* m_wpc;        // [M] words per cell = ceil(n_m / 64)
  const uint32_t* nidx;         // [N] index of node n among its method's nodes
  const uint32_t* mnode_ptr;    // [M+1] CSR of each method's nodes in index order
  const uint32_t* mnodes;
  const uint32_t* mgrow_ptr;    // [Dm+1] CSR of each module's global-row slot gids (ascending)
  const uint32_t* mgrow;
};

// ---- device layout of a batch (layout.cu): the per-node / per-edge part of (a1)
// run as kernels over the uploaded descriptor arrays.  The host validates and lays out only the
// per-type / per-method / per-module tables; node records, operand rows, fact offsets, field-row
// and projection tables, edge records and V1-V6 of every node and edge are computed here.
__host__ __device__ __forceinline__ uint32_t kind_cls(uint32_t k) {
  switch (k) {
    case GK_COPY: case GK_SLOAD: case GK_SSTORE: case GK_RETV: return C_SINGLE;      // (ii)
    case GK_FLOAD: case GK_FSTORE: case GK_ALOAD: case GK_ASTORE: return C_DOUBLE;   // (iii)
    case GK_CALL: return C_CALL;
    case GK_EXIT: return C_EXIT;
    default: return C_ONETIME;                                                      // (i)
  }
}

// Per-app bases of a batch.  Raw per-node arrays are concatenated app after app (node ids, method
// ids, slot gids and node_ops stay app-local in them); row_ptr / call_arg_ptr slices hold n+1
// entries each, so app k's start at node_base + k.
struct __align__(16) DLApp {
  uint64_t key_base;     // dense (module, field) table of the app: key_base + d * n_fields + f
  uint64_t pair_base;    // dense (module, module) table: pair_base + sm * n_mods + dm
  uint64_t n_edges;      // E of the app
  uint32_t node_base, n_nodes, edge_base, arg_base, n_args;
  uint32_t meth_base, n_meths, mod_base, n_mods;
  uint32_t n_fields, n_inst;
  uint32_t stat_lo, stat_hi; // app-local slot gids of the statics: [L_total, L_total + G)
  uint32_t ptr_base;     // = node_base + k (row_ptr / call_arg_ptr slices)
  uint32_t pad[2];
};

// Error word of the layout kernels: min over (app << 44 | node << 4 | code), code = -status.
constexpr unsigned long long DL_NO_ERR = ~0ull;

struct DLDev {
  // uploaded descriptor arrays (app-local values)
  const uint8_t* kind; const uint32_t* meth; const int32_t* ops;
  const uint64_t* rp; const uint64_t* ap; const uint32_t* col; const uint8_t* ekind;
  const int32_t* cargs; const uint32_t* mentry;
  const DLApp* apps; uint32_t n_apps;
  uint32_t N;
  uint64_t K, P;                // entries of the dense key / pair tables of the batch
  // scratch
  uint32_t* words;              // [N] padded block words (scan input)
  uint64_t* foff;               // [N+1] fact offsets (exclusive scan)
  uint32_t* ksz; uint64_t* koff;  // [K] field-row table size (n_cols) of used keys, 0 else; offsets [K+1]
  uint32_t* psz; uint64_t* poff;  // [P] projection table size of used module pairs, 0 else; [P+1]
  uint32_t* cls;                // [NCLS] work items per class
  unsigned long long* err;      // DL_NO_ERR or the first error
  // uploaded per-method / per-module tables (batch-global indices)
  const MethRec* meths; const ModRec* mods;
  const uint32_t* col_gid; const int32_t* col_type; const uint32_t* col_hbase;
  const uint32_t* grow_gid; const uint32_t* tf_ptr; const uint32_t* tf;
  // outputs
  NodeRec* nodes; uint32_t* nodemeth; uint32_t* rowptr; uint32_t* argptr; int32_t* args;
  Edge* edges; InlEdge* inl; int32_t* frow; int32_t* xmap;
};
// phase 1: validate nodes / edges, block sizes, used keys and module pairs, class counts, scans
cudaError_t launch_dl_sizes(const DLDev& L, uint64_t* scan_tmp, cudaStream_t s);
// phase 2 (after the host allocated frow / xmap from the totals): records, tables, edges
cudaError_t launch_dl_records(const DLDev& L, cudaStream_t s);
// totals + error word into mapped pinned host memory (no copy-engine round trip)
cudaError_t launch_dl_totals(const DLDev& L, uint64_t* host_mapped, cudaStream_t s);

int plain_max_blocks(int device);
cudaError_t launch_plain(const PlainDev& P, uint32_t blocks, cudaStream_t s);
cudaError_t launch_plain_digest(const PlainDev& P, cudaStream_t s);
cudaError_t launch_cell_to_mat(const PlainDev& P, const Dev& D, cudaStream_t s);
cudaError_t launch_plain_sizes(const PlainDev& P, uint32_t n0, uint32_t n1, uint64_t* out, cudaStream_t s);
cudaError_t launch_plain_gather(const PlainDev& P, uint32_t n0, uint32_t n1, const uint64_t* ptr, uint64_t* pairs,
                                cudaStream_t s);

// kernels.cu launch wrappers (return cudaError_t of the launch)
cudaError_t launch_seed(const Dev& D, cudaStream_t s);
cudaError_t launch_nmask_rebuild(const Dev& D, cudaStream_t s);
cudaError_t launch_rebase(const Dev& D, NodeRec* nodes, uint32_t* nodemeth, uint32_t* rowptr, uint32_t* argptr,
                          const AppBase* bases, cudaStream_t s);
cudaError_t launch_edges(const Dev& D, Edge* edges, InlEdge* inl, NodeRec* nodes, const uint32_t* ecol,
                         const uint8_t* ekind, const uint32_t* exoff, cudaStream_t s);
cudaError_t launch_fixpoint(const Dev& D, uint32_t blocks, cudaStream_t s);
cudaError_t launch_sbda(const Dev& D, uint32_t blocks, cudaStream_t s);
cudaError_t launch_meth_csr(const Dev& D, uint32_t* ptr, uint32_t* nodes, uint32_t* cursor, cudaStream_t s);
int sbda_max_blocks(int device, uint32_t wide);
cudaError_t launch_round(const Dev& D, uint32_t round, uint32_t blocks, cudaStream_t s);
cudaError_t launch_digest(const Dev& D, cudaStream_t s);
// exclusive prefix of counts[0..n) (u32) into ptr[0..n] (u64) on the device; tmp >= 2 * nblk u64
cudaError_t launch_scan_counts(const uint32_t* counts, uint32_t n, uint64_t* ptr, uint64_t* tmp, cudaStream_t s);
size_t scan_tmp_words(uint32_t n);
cudaError_t launch_popc(const Dev& D, uint32_t n0, uint32_t n1, uint64_t* out, cudaStream_t s,
                        const uint32_t* list = nullptr);
cudaError_t launch_expand(const Dev& D, uint32_t n0, uint32_t n1, const uint64_t* ptr,
                          uint64_t* pairs, cudaStream_t s, const uint32_t* list = nullptr,
                          uint32_t max_blocks = 0);
int fixpoint_max_blocks(int device, uint32_t wide, uint32_t hiocc);

}  // namespace gd
