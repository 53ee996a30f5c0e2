/*
 * oracle.h — C interface of the CPU ORACLE for GDroid's IDFG construction.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load liboracle.so.
 * The product path (paper_conf_ipps_yuwobby20_b200) never links, imports or
 * calls anything here, and this file shares no code or header with it.
 *
 * What it computes: the least fixed point IN(n) of the data-flow equations of
 * SURVEY.md §8(c) C1-C4 by Alg. 1's sequential worklist,
 * over explicit sorted sets of (slot gid, instance gid) pairs — the paper's
 * set representation (Fig. 5a).  Readings of the paper are
 * listed in DESIGN.md §3.
 */
#ifndef GDROID_ORACLE_H
#define GDROID_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* Input arrays (caller-owned, read during oracle_build only).  Field meaning is
 * the synth/icfg.py input format. */
typedef struct {
  uint32_t n_nodes, n_methods, n_modules, n_types, n_instances, n_statics, n_fields, n_entries;
  uint64_t n_edges;
  const uint64_t* row_ptr; const uint32_t* col; const uint8_t* edge_kind;
  const uint8_t* node_kind; const uint32_t* node_method; const int32_t* node_ops;
  const uint64_t* call_arg_ptr; const int32_t* call_args;
  const uint32_t* method_entry; const uint32_t* method_exit; const uint32_t* method_module;
  const uint32_t* method_n_locals; const uint32_t* method_n_params;
  const uint64_t* module_inst_ptr; const uint32_t* module_insts;
  const uint64_t* module_static_ptr; const uint32_t* module_statics;
  const int32_t* inst_type;
  const uint64_t* type_field_ptr; const uint32_t* type_fields;
  const uint32_t* entries;
} oracle_icfg;

typedef struct oracle_result oracle_result;

/* order: 0 = FIFO (Alg. 1), 1 = LIFO, 2 = seeded uniform-random pop, 3 = smallest node id first.
 * Returns 0 on success, -1 invalid structure (V5/V6), -2 pool violation (V1-V4). */
int oracle_build(const oracle_icfg* g, int order, uint64_t seed, oracle_result** out);
void oracle_free(oracle_result* r);
const char* oracle_last_error(void);

uint64_t oracle_visits(const oracle_result* r);
double oracle_seconds(const oracle_result* r);
uint64_t oracle_total_pairs(const oracle_result* r);
/* all IN sets as CSR: ptr[n_nodes+1], pairs[total] = (slot_gid<<32)|inst_gid ascending */
void oracle_all_pairs(const oracle_result* r, uint64_t* ptr, uint64_t* pairs);
/* C8 digests: per_node may be NULL */
void oracle_digests(const oracle_result* r, uint64_t* per_node, uint64_t* app);
/* Post-fixpoint check: number of (edge, pair) violations of T_e(f_p(IN(p))) ⊆ IN(n)
 * over reached p, plus the number of unreached nodes with a non-empty IN. */
uint64_t oracle_check_postfix(const oracle_icfg* g, const oracle_result* r);

/* BSP-round variant (Fig. 2 round sequence): every round pops the
 * whole current list, in order; successors that grew or were never visited form the
 * next list (first insertion order, de-duplicated).  Writes up to cap node ids into
 * seq, and for each round its length into lens (up to lens_cap rounds).
 * Returns the number of rounds, or <0 on error. */
int64_t oracle_bsp_rounds(const oracle_icfg* g, uint32_t* seq, uint64_t cap,
                          uint32_t* lens, uint64_t lens_cap);


/* Fig. 7 MER primitive: given the current worklist wl[0..n) and the
 * destinations dst[0..nd) produced by processing its head list, form the next worklist:
 * head = first floor(n/32)*32 nodes (whole list if n <= 32), next = the
 * destinations not already in the tail (de-duplicated, first occurrence kept) followed by
 * the unprocessed tail — Fig. 7 prints {Nx,...,Ny, N32, N33, N34, N35}.
 * Writes the head size to *head_n and returns the next list length (<= cap). */
uint64_t oracle_mer_merge(const uint32_t* wl, uint64_t n, const uint32_t* dst, uint64_t nd,
                          uint32_t* next, uint64_t cap, uint64_t* head_n);

#ifdef __cplusplus
}
#endif
#endif
