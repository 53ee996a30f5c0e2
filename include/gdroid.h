/*
 * gdroid.h — C ABI of the B200-native IDFG construction library (libgdroid.so).
 *
 * What the library computes: the Inter-procedural Data-Flow Graph of Eq. (1)
 * (PAPER.md:351-355), IDFG(E_C) = ((N,E), {fact(n) | n in N}), by the worklist
 * fixed point of Alg. 1 re-designed as Alg. 3-style device
 * rounds: matrix/bitset facts (MAT, §IV-A),
 * class-grouped worklists (GRP, §IV-B) and de-duplicated
 * merged worklists (MER, §IV-C).  fact(n) is the in-set
 * IN(n) (DESIGN.md §3 reading A4); the exact semantics — node transfer
 * functions, CALL/RET/C2R edge transforms with pool projection — are
 * SURVEY.md §8(c) C1-C4 as restated in DESIGN.md §3.
 *
 * Every entry point is extern "C", takes plain pointers and sizes, never throws,
 * and returns a gdroid_status (negative = error; gdroid_last_error() gives a
 * message naming the first offending index).
 *
 * Ownership: all desc arrays are caller-owned HOST memory, read only during
 * gdroid_load_*; the caller may free them on return.  A gdroid_app handle owns
 * all device and pinned memory it allocates until gdroid_free (which accepts
 * NULL).  Distinct handles may be used concurrently from different threads; a
 * single handle is not thread-safe.
 *
 * Streams: all device work of a handle is issued on the cudaStream_t passed to
 * gdroid_load_* (NULL = legacy default stream).  gdroid_build_idfg is
 * synchronous unless opts->async is set (then gdroid_sync completes it).
 */
#ifndef GDROID_H
#define GDROID_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define GDROID_ABI_VERSION 2u   /* 2: gdroid_build_opts.release_facts, gdroid_release_facts */

typedef enum {
  GDROID_OK = 0,
  GDROID_E_INVALID = -1,  /* structural fault: CSR, ids, edge/node kinds (V5), arity (V6)    */
  GDROID_E_POOL = -2,     /* pool closure violated (V1-V4)                     */
  GDROID_E_OOM = -3,      /* device or pinned allocation failed                             */
  GDROID_E_CUDA = -4,     /* CUDA runtime error (message has the CUDA error string)          */
  GDROID_E_STATE = -5,    /* read before build / sync without a pending async build          */
  GDROID_E_RANGE = -6,    /* node or app index out of range                                  */
  GDROID_E_SMALLBUF = -7, /* caller buffer too small; *n_pairs holds the needed count        */
  GDROID_E_LIMIT = -8     /* max_rounds exceeded (facts are an under-approximation), or a
                             size limit (> 512 instances in one module pool, > 2^32 edges)  */
} gdroid_status;

/* Node kinds: SURVEY §8(c) C2; the paper's 9 statement + 17 expression kinds
 * map onto these (DESIGN.md §3 table). */
typedef enum {
  GK_NOP = 0, GK_ENTRY, GK_EXIT, GK_RETSITE, GK_CALL, GK_PRIM, GK_CONST, GK_NEW,
  GK_COPY, GK_SLOAD, GK_SSTORE, GK_RETV, GK_FLOAD, GK_FSTORE, GK_ALOAD, GK_ASTORE
} gdroid_node_kind;

/* Edge kinds: SURVEY §8(c) C3 ("blue arrow-lines", Fig. 2). */
typedef enum { GE_INTRA = 0, GE_CALL, GE_RET, GE_C2R } gdroid_edge_kind;

#define GDROID_F_ARR 0u   /* the array pseudo-field id */

typedef struct gdroid_app gdroid_app;   /* opaque; owns device memory */

/* One app's ICFG (Alg. 2 l.1 h_icfg/h_stmt) plus the
 * pre-determined slot and instance pools.
 * Slot gids: locals method-major (local_base[m] + i, params first, RET last),
 * then statics (L_total + g), then heap slots
 * (L_total + n_statics + heap_base[o] + ordinal of f in F(t(o))). */
typedef struct {
  uint32_t abi_version;      /* must be GDROID_ABI_VERSION */
  uint32_t n_nodes, n_methods, n_modules, n_types, n_instances, n_statics, n_fields, n_entries;
  uint64_t n_edges;
  const uint64_t* row_ptr;   /* [n_nodes+1] CSR over node ids                               */
  const uint32_t* col;       /* [n_edges]   successor node id                               */
  const uint8_t*  edge_kind; /* [n_edges]   gdroid_edge_kind                                */
  const uint8_t*  node_kind; /* [n_nodes]   gdroid_node_kind                                */
  const uint32_t* node_method;/* [n_nodes]                                                  */
  const int32_t*  node_ops;  /* [n_nodes*4] {op0 lhs slot gid, op1 rhs slot gid, op2 field,
                                op3 instance gid | RETSITE: its CALL node}; -1 = none.
                                FLOAD v=w.f: op0=v, op1=w.  FSTORE v.f=w: op0=v, op1=w.
                                SSTORE g=w: op0=g.  RETV w: op1=w.  CALL/RETSITE: op0=lhs. */
  const uint64_t* call_arg_ptr;/* [n_nodes+1] CSR of actual args per CALL node             */
  const int32_t*  call_args; /* local slot gid of the actual, -1 = non-reference actual      */
  const uint32_t* method_entry, *method_exit, *method_module, *method_n_locals, *method_n_params;
  const uint64_t* module_inst_ptr; const uint32_t* module_insts;     /* sorted, contains 0 */
  const uint64_t* module_static_ptr; const uint32_t* module_statics; /* sorted static ids  */
  const int32_t*  inst_type;  /* [n_instances]; -1 only for instance 0 = NULL              */
  const uint64_t* type_field_ptr; const uint32_t* type_fields;       /* sorted field ids   */
  const uint32_t* entries;    /* [n_entries] ENTRY nodes of component environment methods  */
} gdroid_icfg_desc;

/* Build options; an all-zero struct (or NULL) means defaults. */
typedef struct {
  uint32_t async;        /* 1: enqueue only, complete with gdroid_sync.  The light/heavy
                            hand-overs of large narrow batches are decided
                            on the device, so nothing in a build waits on the host.        */
  uint32_t max_rounds;   /* 0 = unlimited                                                   */
  uint32_t blocks;       /* persistent-kernel CTAs (0 = SMs x occupancy)                     */
  uint32_t loop_mode;    /* 0 = persistent cooperative kernel (default), 1 = host-launched
                            round kernels (one launch per round)                            */
  uint32_t variant;      /* gdroid_variant: ablation of the paper's optimisations (SURVEY
                            §8(f) 1).  Every variant computes the same
                            least fixed point; only the schedule / data structure differ.  */
  uint32_t no_byte_model;/* 1: skip the on-device byte-model counters (alg_bytes, dense_bytes
                            and atomics of the stats are then 0); rounds and visits are
                            always counted.  A separate kernel instantiation without the
                            counting code (fewer instructions per visit).                  */
  uint32_t release_facts;/* 1: after the digests, return the fact store to the device's
                            stream-ordered memory pool (gdroid_release_facts); the digests
                            stay readable, the facts do not (GDROID_E_STATE) until the next
                            build re-allocates and rebuilds them.  Lets a corpus keep every
                            app's tables resident while only the batch being built holds a
                            fact store.                                       */
  uint32_t keep_facts;   /* 1: incremental build: the fact store keeps its
                            content (an earlier build of this handle, or gdroid_import_facts),
                            the worklist history persists, and the first round queues only
                            the seeds staged with gdroid_stage_seeds (plus the entries on the
                            handle's first build).  IN only grows, so this continues the same
                            monotone iteration: the out-of-core sub-graph loop (§III-A1,
                            PAPER.md:524-580) runs each sub-graph this way until no seed
                            changes.                                                         */
  uint32_t reserve_sms;  /* leave this many SMs' worth of CTAs out of the persistent grid, so
                            kernels on other streams (e.g. the fact readback of the previous
                            batch) run beside the fixed point; 0 = full grid */
} gdroid_build_opts;

/* Variants (Fig. 8-12), recast on B200:
 *   DEFAULT  the B200 path: MAT + GRP + round-stamp dedupe + continuation into wide successors
 *   MAT      matrix store (MAT); one worklist segment in arrival order; no
 *            head/tail merging; no continuation
 *   MAT_GRP  + class-segmented worklists (GRP)
 *   GDROID   + MER: each round processes the head list (whole waves of the grid's warps) and
 *            merges the tail into the next worklist (Fig. 7)
 *   PLAIN    the set-based plain implementation (Alg. 2): per-node sorted
 *            pair arrays with regrowth from a device bump allocator, one thread per node,
 *            per-thread switch over node kinds; needs a handle loaded with
 *            gdroid_load_icfg_plain (one app)
 *   CELL     the paper's own MAT layout (Fig. 5b): one
 *            cell-major matrix per method (rows = the method's slot pool, columns = its
 *            instance pool, cell = an n_m-bit mask over the method's statements), run by the
 *            PLAIN schedule (thread per node: IN(n) gathered from bit n of every cell, unions
 *            = one atomicOr per pair); the facts are converted to the node-major store for
 *            readback.  Needs a gdroid_load_icfg_plain handle; fact_bytes = the cell store.
 *   SBDA     the paper's two-level decomposition (§III-A2, Fig. 3; Alg. 2
 *            l.6 mid <- blockIdx.x): per pass, every method with queued nodes is claimed by
 *            one CTA, which runs that method's worklist to local quiescence in shared memory
 *            (__syncthreads between local rounds); CALL / RET successors start the next pass.
 *            Same least fixed point (DESIGN.md §5.6 and reading R8); rounds = passes.        */
typedef enum { GDROID_V_DEFAULT = 0, GDROID_V_MAT = 1, GDROID_V_MAT_GRP = 2, GDROID_V_GDROID = 3,
               GDROID_V_PLAIN = 4, GDROID_V_CELL = 5, GDROID_V_SBDA = 6 } gdroid_variant;

/* Device-counted statistics of the last build (DESIGN.md §5 byte models). */
typedef struct {
  uint64_t rounds;        /* worklist iterations (device rounds)                            */
  uint64_t node_visits;   /* nodes processed, summed over rounds (Alg. 1 pops)               */
  uint64_t alg_bytes;     /* touched-word byte model, summed over visits     */
  uint64_t dense_bytes;   /* dense MAT byte model, summed over visits                        */
  uint64_t atomics;       /* 64-bit atomicOr issued into successor in-sets                   */
  uint64_t hist[3];       /* rounds with frontier <= 32, 33..64, > 64 (Table II buckets)     */
  uint64_t build_ns;      /* CUDA-event time of the build (zero + fixed point + digest)      */
  uint64_t fixpoint_ns;   /* CUDA-event time of the fixed-point kernel(s) alone              */
  uint64_t h2d_ns;        /* host time of the load's upload                                  */
  uint64_t fact_bytes;    /* size of the device fact store                                   */
  uint64_t kernel_launches; /* kernels launched by the last build                            */
} gdroid_build_stats;

/* Load one app (= a batch of one). */
gdroid_status gdroid_load_icfg(const gdroid_icfg_desc* desc, int device, void* cuda_stream,
                               gdroid_app** out);
/* Load n_apps independent apps into ONE handle; they share every device round
 * (IDFG-instance batching).  Node ids, slot gids and digests stay
 * per app.  Device layout (the default): the host validates and lays
 * out only the per-type / per-method / per-module tables (apps in parallel on a worker
 * pool of min(hardware threads, $GDROID_HOST_THREADS) threads), copies the raw
 * descriptor arrays into a pinned staging buffer and uploads them; kernels resolve the
 * operands, validate every node and edge (V1-V6), and build the node / edge records and
 * the field-row and projection tables.  The call waits for those kernels (two short
 * round trips), so every validation error is returned by this call: the host validator
 * then re-runs for the exact status and message.  $GDROID_HOST_LAYOUT=1 (and hosts
 * without a device) lay out every table on the host instead (same bytes).  The
 * descriptor arrays are only read during the call. */
gdroid_status gdroid_load_batch(const gdroid_icfg_desc* descs, uint32_t n_apps, int device,
                                void* cuda_stream, gdroid_app** out);
/* Load ONE app for every variant including GDROID_V_PLAIN: the MAT handle of
 * gdroid_load_icfg plus device copies of the descriptor arrays and the set-based
 * state of the plain variant (per-node pair arrays in a bump-allocated heap sized
 * from the pools' dense bound, per-thread scratch).
 * Readback after a PLAIN build returns the sets; digests are computed from them. */
gdroid_status gdroid_load_icfg_plain(const gdroid_icfg_desc* desc, int device, void* cuda_stream,
                                     gdroid_app** out);
/* Zero the fact store, seed the entries, run the fixed point, compute digests. */
gdroid_status gdroid_build_idfg(gdroid_app* app, const gdroid_build_opts* opts,
                                gdroid_build_stats* stats);
gdroid_status gdroid_sync(gdroid_app* app, gdroid_build_stats* stats);
/* ---- incremental builds and out-of-core sub-graphs ----
 * Stage seeds for the next keep_facts build of app k: for each of the n nodes (app-local ids),
 * the pairs pairs[ptr[i] .. ptr[i+1]) (slot_gid << 32 | inst_gid, the app's gids) are OR-ed
 * into IN(node) and the node is queued even if it gets no pair (first reach, reading A5).
 * Arrays are read during the call.  A pair outside the node's pools makes that build return
 * GDROID_E_POOL. */
gdroid_status gdroid_stage_seeds(gdroid_app* app, uint32_t k, uint32_t n, const uint32_t* nodes,
                                 const uint64_t* ptr, const uint64_t* pairs);
/* Facts of the listed nodes of app k (app-local ids): ptr[n+1] and pairs, two-call like
 * gdroid_read_all_facts (the boundary proxies of out-of-core sub-graphs). */
gdroid_status gdroid_read_nodes_facts(const gdroid_app* app, uint32_t k, uint32_t n,
                                      const uint32_t* nodes, uint64_t* ptr, uint64_t* pairs,
                                      uint64_t cap);
/* out[i] = 1 if node nodes[i] of app k was ever queued (reached) by the builds so far. */
gdroid_status gdroid_read_reached(const gdroid_app* app, uint32_t k, uint32_t n,
                                  const uint32_t* nodes, uint8_t* out);
/* Raw copies of the whole device fact store (gdroid_fact_bytes bytes, the library's own
 * layout) to / from caller host memory, enqueued on the handle's stream (pinned memory: an
 * asynchronous DMA; complete with gdroid_stream_sync).  Import re-allocates a released store;
 * a keep_facts build then continues from the imported facts. */
gdroid_status gdroid_export_facts(const gdroid_app* app, void* host, uint64_t bytes);
gdroid_status gdroid_import_facts(gdroid_app* app, const void* host, uint64_t bytes);
gdroid_status gdroid_stream_sync(gdroid_app* app);
uint64_t      gdroid_fact_bytes(const gdroid_app* app);
/* Free the handle's fact store (stream-ordered, cudaFreeAsync on the handle's stream; the
 * library raises the device pool's release threshold so the memory stays reserved for the
 * next allocation).  Tables, digests and stats remain; gdroid_read_* return GDROID_E_STATE
 * until the next gdroid_build_idfg, which re-allocates the store.  Idempotent. */
gdroid_status gdroid_release_facts(gdroid_app* app);
/* Facts of one node of app k as strictly ascending (slot_gid << 32 | inst_gid).
 * pairs == NULL: size query.  cap < needed: GDROID_E_SMALLBUF with *n_pairs set. */
gdroid_status gdroid_read_facts(const gdroid_app* app, uint32_t node, uint64_t* pairs,
                                uint64_t cap, uint64_t* n_pairs);
gdroid_status gdroid_read_facts_in(const gdroid_app* app, uint32_t k, uint32_t node,
                                   uint64_t* pairs, uint64_t cap, uint64_t* n_pairs);
/* All facts of app k: ptr[n_nodes+1] and pairs (two-call: pairs == NULL fills ptr only). */
gdroid_status gdroid_read_all_facts(const gdroid_app* app, uint32_t k, uint64_t* ptr,
                                    uint64_t* pairs, uint64_t cap);
/* All facts of EVERY app of the batch as one CSR over the batch's nodes in load order (app k
 * owns rows sum_{j<k} n_nodes(j) ..): ptr[N_batch+1], pairs as in gdroid_read_all_facts (each
 * app in its own slot / instance gids).  Two-call: pairs == NULL fills ptr only (the per-node
 * counts stay on the device for the fetch).  Pinned caller buffers give full-rate copies
 * (Alg. 3 l.17 h_fact <- d_fact_mat). */
gdroid_status gdroid_read_batch_facts(const gdroid_app* app, uint64_t* ptr, uint64_t* pairs,
                                      uint64_t cap);
/* Asynchronous form of gdroid_read_batch_facts: scans the offsets on the device
 * (one 8-byte synchronous copy of the pair count into *total), expands the pairs on the device
 * and enqueues the copies of ptr[N_batch+1] and of the pairs into the caller's PINNED buffers
 * without waiting, so they overlap the next work enqueued (the next batch's fixed point).
 * Complete with gdroid_stream_sync; the buffers must stay valid until then.  *total > cap:
 * GDROID_E_SMALLBUF, nothing copied.  `blocks` is reserved (0). */
gdroid_status gdroid_read_batch_facts_async(gdroid_app* app, uint64_t* ptr, uint64_t* pairs,
                                            uint64_t cap, uint64_t* total, uint32_t blocks);
/* Per-node digests d(n) = sum over IN(n) of mix64(mix64(n) ^ pair),
 * computed on the device at the end of the build; per_node may be NULL. */
gdroid_status gdroid_node_digests(const gdroid_app* app, uint64_t* per_node, uint64_t* app_digest);
/* The same for app k of a batch: per_node[n_nodes(k)] indexed by the app's own node ids. */
gdroid_status gdroid_node_digests_in(const gdroid_app* app, uint32_t k, uint64_t* per_node,
                                     uint64_t* app_digest);
gdroid_status gdroid_app_digests(const gdroid_app* app, uint64_t* per_app /* [n_apps] */);
uint32_t      gdroid_n_apps(const gdroid_app* app);
/* Diagnostics: record a per-round trace in the next builds (cap rounds, 0 = off), then read
 * it back as pairs {globaltimer ns at round start, items << 32 | nodes}; *n = rounds recorded
 * (the last entry, with 0 items, marks the end of the fixed point). */
gdroid_status gdroid_debug_trace(gdroid_app* app, uint32_t cap);
gdroid_status gdroid_debug_read_trace(const gdroid_app* app, uint64_t* out, uint64_t cap, uint64_t* n);
/* Diagnostics: per-phase cycle counters of the last build (only filled by a library compiled
 * with -DGD_PHASES): setup, edges, pushes, round end (publish + grid barrier), items. */
gdroid_status gdroid_debug_phases(const gdroid_app* app, uint64_t* out8);
/* Diagnostics: copy one of the handle's device tables to host memory, to compare
 * the device layout (layout.cu, the default) with the host layout ($GDROID_HOST_LAYOUT=1) byte for
 * byte.  which: 0 NodeRec[N] (64 B), 1 Edge[E] (32 B), 2 InlEdge[4N] (16 B), 3 field-row table
 * (i32), 4 projection tables (i32), 5 argument rows (i32), 6 row_ptr u32[N+1], 7 arg_ptr
 * u32[N+1], 8 node-method u32[N].  host == NULL: *bytes = the size only; cap < size:
 * GDROID_E_SMALLBUF. */
gdroid_status gdroid_debug_tables(const gdroid_app* app, uint32_t which, void* host, uint64_t cap,
                                  uint64_t* bytes);
void          gdroid_free(gdroid_app* app);
const char*   gdroid_last_error(void);   /* thread-local; valid until the next call */
uint32_t      gdroid_abi_version(void);

#ifdef __cplusplus
}
#endif
#endif
