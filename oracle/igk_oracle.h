/*
 * igk_oracle.h -- CPU oracle for the iG-kway incremental refinement step.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load this library.
 * The product path (paper_conf_dac_leejlczcshh25_b200/) never includes,
 * links or calls anything under oracle/, and this file shares no header,
 * constant or helper with include/igk.h.
 *
 * Semantics: IGK-SEM v1, i.e. the paper's
 * Alg. 1-4 (PAPER.md P:94-P:270) read under the fixed readings listed in
 * DESIGN.md section 4.  A plain, single-threaded, slow implementation on
 * flat arrays; every function cites the passage it follows.
 *
 * Pins (tests/test_oracle_pins.py): worked examples, exact-rational cap,
 * brute-force step replay, exhaustive optimum, invariants.  R3 (balance
 * restoration) follows reading Q9 of a passage the paper leaves silent: its
 * implementation is pinned by brute force, but the reading itself is
 * "parity unpinned" against the paper.
 *
 * Modifiers are passed as int32 quadruples {kind, u, v, w}:
 *   kind 0 = edge deletion  M-(u,v)
 *   kind 1 = vertex deletion M-u      (Alg. 2)
 *   kind 2 = vertex insertion M+u     (Alg. 2); w = vertex weight
 *   kind 3 = edge insertion  M+(u,v)  (Alg. 1); w = edge weight
 */
#ifndef IGK_ORACLE_H
#define IGK_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct ora_graph ora_graph;

/* return codes (numerically equal to the product's, by specification) */
#define ORA_OK 0
#define ORA_EINVAL 1
#define ORA_ENOMEM 2
#define ORA_ESTATE 5
#define ORA_WIMBALANCED 6

/* stats vector layout (ORA_NSTATS int64 entries) */
enum {
  ORA_ST_AFFECTED = 0,   /* |A u Psi0|: directly affected (A) + pending inserted */
  ORA_ST_INSERTED,       /* |Psi0|: pending pseudo vertices at refine start      */
  ORA_ST_EXPANDED,       /* |N|: non-pseudo neighbours of Psi examined in R2     */
  ORA_ST_FILTERED_IN,    /* |C1|                                                  */
  ORA_ST_EXPANDED_IN,    /* |C2|                                                  */
  ORA_ST_EVICTED,        /* |R3 evictions|                                        */
  ORA_ST_ROUNDS,         /* R                                                     */
  ORA_ST_MOVES_APPLIED,  /* sum L_r                                               */
  ORA_ST_MOVES_DEFERRED, /* sum (|S_r| - L_r)                                     */
  ORA_ST_CUT,            /* cut after refine                                      */
  ORA_ST_CAP,            /* c = cap(W)                                            */
  ORA_ST_MAX_PART_WEIGHT,
  ORA_ST_IMBALANCED,     /* 1 if the weighted fallback fired                      */
  ORA_NSTATS
};

ora_graph* ora_create(int64_t n, const int64_t* xadj, const int32_t* adjncy,
                      const int32_t* vwgt, const int32_t* adjwgt, int32_t k,
                      double epsilon, const int32_t* init_part, int* status);
void ora_destroy(ora_graph* g);
const char* ora_last_error(const ora_graph* g);

int ora_apply(ora_graph* g, const int32_t* mods, int64_t count,
              int64_t* first_new_id, int64_t* bad_index);
int ora_refine(ora_graph* g, int64_t* stats /* ORA_NSTATS, nullable */);
/* NEXT-1: A |= every boundary vertex (adj_ext != 0), then refine */
int ora_refine_global(ora_graph* g, int64_t* stats /* ORA_NSTATS, nullable */);
/* NEXT-2 full repartition of the current graph ("applications can
 * resort to FGP ... when the number of graph modifiers reaches 50% of the
 * graph's size"), reading F8: the active vertices relabelled
 * densely in ID order, their induced graph (rows ascending) partitioned by
 * ora_fgp with the handle's k and epsilon, the parts written back; deleted
 * vertices stay deleted.  ORA_ESTATE if a batch is applied but not refined
 * (pending affected or pseudo vertices); the I4 baseline restarts. */
int ora_repartition(ora_graph* g, int32_t group_size);

int64_t ora_n_total(const ora_graph* g);
int64_t ora_n_active(const ora_graph* g);
/* out[v] = part, -1 = deleted, -2 = pending (pseudo) */
void ora_partition(const ora_graph* g, int32_t* out);
int64_t ora_cut(const ora_graph* g);             /* recount from scratch */
void ora_part_weights(const ora_graph* g, int64_t* out_k);
int64_t ora_total_weight(const ora_graph* g);
int64_t ora_cap_value(const ora_graph* g);
/* symmetric CSR of the current graph over all IDs, rows sorted ascending */
int64_t ora_num_slots(const ora_graph* g);
void ora_export_csr(const ora_graph* g, int64_t* xadj, int32_t* adjncy, int32_t* adjwgt);
/* invariants I1-I6; returns 0 if all hold, else writes msg
 * (tagged "I6: ...", "I5: ...", ...: the first violation in the order
 * I6, I5, I2, I3, I4, I1).  I1 compares reported_cut (e.g. the maintained
 * cut of the product) with the recount; reported_cut < 0 skips I1.
 * flags & 1 skips the O(m log m) structural check I6. */
int ora_check_invariants_ext(const ora_graph* g, int64_t reported_cut, int flags, char* msg, int msglen);
int ora_check_invariants(const ora_graph* g, char* msg, int msglen);

/* TEST-ONLY corruption hooks (pins of the invariant checker): each writes
 * one field of the state; p < 0 in set_part means the pseudo label */
void ora_debug_set_part(ora_graph* g, int64_t v, int32_t p);
void ora_debug_set_part_weight(ora_graph* g, int32_t p, int64_t w);
void ora_debug_set_total_weight(ora_graph* g, int64_t W);
void ora_debug_set_frontier(ora_graph* g, int64_t v, int f);
void ora_debug_add_half_edge(ora_graph* g, int64_t u, int32_t x, int32_t w);
void ora_debug_set_edge_weight(ora_graph* g, int64_t u, int32_t x, int32_t w);

/* wide = 1: coarse-level graphs of the full partitioner (vertex / edge
 * weights up to INT32_MAX, totals <= INT32_MAX, no modifiers accepted) */
ora_graph* ora_create_ex(int64_t n, const int64_t* xadj, const int32_t* adjncy,
                         const int32_t* vwgt, const int32_t* adjwgt, int32_t k,
                         double epsilon, const int32_t* init_part, int wide, int* status);

/* NEXT-2: IGK-FGP v1 full partitioning (igk_fgp.c):
 * constrained coarsening (group size s), greedy initial partition of the
 * coarsest graph, projection + global boundary refinement per level.
 * part_out[n]; level_n[l] = vertices of level l (up to maxlev entries).
 * Returns the number of levels (>= 1) or -ORA_EINVAL. */
int ora_fgp(int64_t n, const int64_t* xadj, const int32_t* adjncy, const int32_t* vwgt,
            const int32_t* adjwgt, int32_t k, double epsilon, int32_t group_size,
            int32_t* part_out, int64_t* level_n, int64_t maxlev);
/* one coarsening step (selection, join labels, groups) of a CSR graph:
 * returns the number of groups; sel/root/label/cmap per vertex */
/* test-only knobs of ora_fgp: refinement passes per level (default 8; 0 =
 * none, the projected initial partition) and the initial partition (0 = BFS
 * graph growing, the default; 1 = contiguous ID blocks) */
void ora_fgp_set_passes(int passes);
void ora_fgp_set_init(int mode);
/* test-only: label-propagation passes per finer level (default 16) */
void ora_fgp_set_lp_passes(int passes);
/* one label-propagation pass (reading F7) on a CSR graph: part updated in
 * place, returns the number of vertices moved, *dcut = the cut reduction */
int64_t ora_fgp_lp_pass(int64_t n, const int64_t* xadj, const int32_t* adjncy, const int32_t* vwgt,
                        const int32_t* adjwgt, int32_t k, double epsilon, int32_t* part, int64_t* dcut);
int64_t ora_fgp_coarsen_step(int64_t n, const int64_t* xadj, const int32_t* adjncy,
                             const int32_t* adjwgt, int32_t group_size, int32_t* sel,
                             int32_t* root, int32_t* label, int32_t* cmap, int64_t* coarsenable);

/* step-level hooks used by the pinning tests (tests/test_oracle_*.py) */
int64_t ora_cap(int64_t W, double epsilon, int32_t k);
/* last refine trace: per round |S_r| and L_r (up to maxr rounds) */
int64_t ora_trace_rounds(const ora_graph* g, int64_t* S, int64_t* L, int64_t maxr);
/* last refine: the sorted move list of every round, (u, p*, g) triples
 * concatenated in round order; returns the number of moves */
int64_t ora_trace_moves(const ora_graph* g, int64_t* out, int64_t cap3);
/* last refine sets: which vertices entered Psi in R1, R2, R3 (flags per ID) */
void ora_trace_sets(const ora_graph* g, uint8_t* c1, uint8_t* c2, uint8_t* r3);

#ifdef __cplusplus
}
#endif
#endif
