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
constexpr int CNT_STRIDE = 8;      // counts[rot * CNT_STRIDE + cls]
constexpr int THREADS = 256;       // fixed-point kernel block size
constexpr int WARPS = THREADS / 32;

// One ICFG node (32 B, one sector).  Row indices r* are relative to the node's fact block
// (method-local rows first, then the module's global rows), resolved by the loader.
struct __align__(16) NodeRec {
  uint64_t off;      // word offset of IN(n) in the fact store
  uint32_t method;   // global method index
  uint8_t kind;      // gdroid_node_kind
  uint8_t cls;       // Cls
  uint16_t app;      // index of the app inside a batch
  int32_t r0;        // lhs row (PRIM/CONST/NEW/COPY/SLOAD/RETV/FLOAD/ALOAD), static row (SSTORE),
                     // base row (FSTORE/ASTORE), lhs row of the call (CALL/RETSITE) or -1
  int32_t r1;        // rhs row (COPY/SLOAD/SSTORE/RETV), w row (FLOAD/ALOAD/FSTORE/ASTORE)
  int32_t r2;        // field id (FLOAD/FSTORE; F_ARR for ALOAD/ASTORE)
  int32_t r3;        // instance column (CONST/NEW)
};
static_assert(sizeof(NodeRec) == 32, "NodeRec must be 32 bytes");

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

struct Edge {
  uint32_t dst;
  uint32_t info;       // kind (2 bits) | xlate id << 2 (0 = same module / identity)
};

struct XRec {          // cross-module projection π (CALL/RET edges between modules)
  uint32_t colmap_off; // colmap[c_src] -> c_dst or -1, |Q_src| entries
  uint32_t rowmap_off; // rowmap[g_dst] -> g_src or -1, n_glob(dst) entries
  uint32_t src_mod, dst_mod;
};

struct DevStats {
  unsigned long long rounds, visits, alg_bytes, dense_bytes, atomics, hist[3], limit_hit, pad;
};

struct Dev {
  const NodeRec* nodes;
  const MethRec* meths;
  const ModRec* mods;
  const XRec* xrecs;
  const uint32_t* row_ptr;
  const Edge* edges;
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
  const int32_t* colmap;
  const int32_t* rowmap;
  const uint32_t* app_node_base;
  const uint32_t* entries;      // global node ids of all component entries of all apps
  uint64_t* facts;
  uint32_t* stamp;              // [N] last round a node was queued for (0 = never)
  uint32_t* queue;              // [3][N] rotating class-segmented worklists
  uint32_t* counts;             // [3][CNT_STRIDE]
  DevStats* stats;
  uint32_t* bar;                // grid barrier {count, generation}
  uint64_t* node_digest;        // [N]
  unsigned long long* app_digest; // [n_apps]
  uint64_t n_words;             // fact store size in words
  uint32_t n_nodes;
  uint32_t n_entries;
  uint32_t seg[NCLS + 1];       // class segment starts inside one queue
  uint32_t max_rounds;
};

// kernels.cu launch wrappers (return cudaError_t of the launch)
cudaError_t launch_seed(const Dev& D, cudaStream_t s);
cudaError_t launch_fixpoint(const Dev& D, uint32_t blocks, cudaStream_t s);
cudaError_t launch_round(const Dev& D, uint32_t round, uint32_t blocks, cudaStream_t s);
cudaError_t launch_digest(const Dev& D, cudaStream_t s);
cudaError_t launch_popc(const Dev& D, uint32_t n0, uint32_t n1, uint64_t* out, cudaStream_t s);
cudaError_t launch_expand(const Dev& D, uint32_t n0, uint32_t n1, const uint64_t* ptr,
                          uint64_t* pairs, cudaStream_t s);
int fixpoint_max_blocks(int device);

}  // namespace gd
