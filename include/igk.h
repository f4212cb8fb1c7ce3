/*
 * igk.h -- C ABI of the B200-native iG-kway incremental refinement library
 *          (libigk.so, hand-written CUDA for sm_100a).
 *
 * The operation is the incremental step of iG-kway (Lee et al., DAC'25;
 * "P:N" = line N of the paper text): apply a batch of graph modifiers to a
 * GPU-resident graph (Sec. V.B, Alg. 1-2), then refine the k-way
 * partition over the affected vertices only (Sec. V.C, Alg. 3-4) until
 * every part weight is <= W_pmax with a low cut.  The exact,
 * deterministic semantics (IGK-SEM v1) and every reading of a garbled or
 * silent passage are in DESIGN.md sections 3-4; results are bit-identical
 * to the CPU oracle under oracle/ (which shares no code with this library).
 *
 * Conventions (all functions):
 *  - Host pointers are read (or written) before the call returns and are
 *    never retained; the caller owns them.  Device pointers (only in the
 *    *_device variants) must stay valid until the call returns.
 *  - Calls are synchronous with respect to host buffers; device work runs
 *    on igk_options.stream (NULL = the legacy default stream).
 *  - Errors: IGK_EINVAL leaves the handle unchanged.  A CUDA error poisons
 *    the handle: every later call returns IGK_ESTATE.  No C++ exception
 *    crosses this boundary.  igk_last_error() describes the last failure.
 *  - One handle per host thread at a time.
 */
#ifndef IGK_H
#define IGK_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct igk_graph igk_graph; /* opaque; owns all device memory */

typedef enum {
  IGK_OK = 0,
  IGK_EINVAL = 1,       /* invalid argument or invalid modifier batch (state unchanged) */
  IGK_ENOMEM = 2,       /* vertex or adjacency capacity exhausted / allocation failed   */
  IGK_ECUDA = 3,        /* CUDA error; the handle is poisoned                            */
  IGK_ENCCL = 4,        /* a collective of a sharded handle failed; the handle is poisoned */
  IGK_ESTATE = 5,       /* handle poisoned by an earlier CUDA error, or NULL handle      */
  IGK_WIMBALANCED = 6   /* result valid, but a weighted corner case left W_p > cap (Q8)  */
} igk_status;

/* modifier kinds: M-(u,v), M-u, M+u, M+(u,v) */
enum {
  IGK_EDGE_DELETE = 0,
  IGK_VERTEX_DELETE = 1,
  IGK_VERTEX_INSERT = 2,
  IGK_EDGE_INSERT = 3
};

/* One modifier, 16 bytes.  Edges are undirected: one modifier per edge; the
 * store keeps both directions (the paper lists both, Fig. 4 caption P:90).
 * w = edge weight (EDGE_INSERT) or vertex weight (VERTEX_INSERT); ignored
 * otherwise.  On a handle created without vwgt (resp. adjwgt) the vertex
 * (resp. edge) weight of an insertion must be 1. */
typedef struct {
  int32_t kind, u, v, w;
} igk_modifier;

/* Host-side collective for sharded handles without NCCL (tests: gloo over
 * torch.distributed; also any MPI-like transport).  allreduce: in-place
 * all-reduce over all ranks of `count` elements at `buf` (HOST memory);
 * dtype 0 = int64, 1 = uint32; op 0 = sum, 1 = min, 2 = max; returns 0 on
 * success.  Every rank calls it in the same order with the same count. */
typedef struct {
  void* ctx;
  int32_t (*allreduce)(void* ctx, void* buf, int64_t count, int32_t dtype, int32_t op);
} igk_comm;

typedef struct {
  int device;              /* CUDA device ordinal                                         */
  void* stream;            /* cudaStream_t; NULL = default stream                          */
  int64_t max_vertices;    /* vertex-ID capacity (0 = 2 n + 65536)                        */
  int64_t max_slots;       /* adjacency slab capacity in entries (0 = 4 x initial + 2^22)  */
  int32_t slack_min;       /* minimum spare slots per vertex (0 = 2), cf. gamma      */
  int32_t validate;        /* reserved: batches are always validated                       */
  int32_t check_invariants;/* 1 = recount cut/W_p after every refine and compare (slow)    */
  int32_t blocks_per_sm;   /* persistent-kernel CTAs per SM (0 = auto)                     */
  /* Vertex-range sharding.  nranks > 1: this
   * handle is rank `rank` of a sharded graph, one process per GPU, all
   * ranks calling every entry point in the same order with the same
   * arguments (collective calls).  Rank r owns the IDs [r B, (r+1) B) of the
   * created graph (B = ceil(n / nranks)) and every r-th inserted ID, stores
   * the adjacency of its vertices plus the entries of other vertices that
   * point at them (ghost prefixes), and keeps labels, weights, W_p
   * replicated.  Each refine exchanges fixed-size all-reduces: the candidate
   * bitmaps of R1/R2, the restoration keys, and per round the move records
   * of the selected vertices -- results are bit-identical to one
   * GPU and to the oracle.  The transport is NCCL (nccl_id: an ncclUniqueId
   * of 128 bytes from igk_nccl_unique_id, shared by all ranks; the library
   * creates its communicator on `device`) or the host callback `comm`. */
  int32_t nranks;          /* 0 or 1 = one GPU                                            */
  int32_t rank;
  const void* nccl_id;     /* ncclUniqueId (128 bytes) or NULL                            */
  const igk_comm* comm;    /* host-callback transport (used when nccl_id == NULL)         */
  /* NEXT-3 (sharded handles): p2p = 1 runs all rounds of a refine in ONE
   * persistent kernel per rank that stores the move records straight into
   * every rank's buffer (peer memory: NVLink P2P between GPUs -- CUDA IPC
   * across processes, direct pointers inside one process -- or the same
   * device) and synchronises the ranks with a device-side barrier, instead
   * of a host round trip + all-reduce per round.  Set up collectively at
   * create (the buffers' addresses / IPC handles are exchanged through the
   * transport).  ranks_per_device > 1 when several ranks share one GPU
   * (tests): each rank's persistent kernel then takes that fraction of the
   * SMs so all of them are resident at once. */
  int32_t p2p;
  int32_t ranks_per_device;
  /* wide_weights = 1: vertex / edge weights up to INT32_MAX with the total
   * vertex weight and the total edge weight <= INT32_MAX (every per-vertex
   * sum of the refine then stays exact in 32 bits) -- the coarse graphs of
   * the full partitioner (igk_fgp_partition).  Such a handle refines but
   * accepts no modifiers (IGK_EINVAL); single GPU only. */
  int32_t wide_weights;
  /* NEXT-2 fallback policy ("applications can resort to FGP ...
   * especially when the number of graph modifiers reaches 50% of the
   * graph's size"; reading F9): fgp_fallback_ppm > 0 makes
   * every successful refine / step check the modifiers accepted since the
   * last full partition (create or repartition); once they reach
   * fgp_fallback_ppm / 1e6 of the active vertices counted then, the call
   * ends with igk_repartition(g, 6) and stats->repartitioned = 1.
   * 0 = off (default).  Single-GPU handles only. */
  int64_t fgp_fallback_ppm;
} igk_options;

typedef struct {
  int64_t affected;        /* |A u Psi0|: directly affected vertices + pending inserts */
  int64_t inserted;        /* |Psi0|: pending pseudo vertices at refine start (Alg. 3 L2-5)  */
  int64_t expanded;        /* |N|: neighbours of pseudo vertices examined in R2      */
  int64_t filtered_in;     /* |C1|: affected vertices moved to the pseudo-partition (R1)     */
  int64_t expanded_in;     /* |C2| (R2)                                                      */
  int64_t evicted;         /* R3 balance-restoration evictions                               */
  int64_t rounds;          /* R: Alg. 4 rounds until the pseudo-partition is empty   */
  int64_t moves_applied;   /* sum of the balanced prefixes L_r                                */
  int64_t moves_deferred;  /* sum of |S_r| - L_r                                              */
  int64_t cut;             /* cut size after the refine                                */
  int64_t cap;             /* c = cap(W) used by this refine (reading Q4)               */
  int64_t max_part_weight;
  int64_t imbalanced;      /* 1 iff the weighted fallback fired (IGK_WIMBALANCED)             */
  int64_t adj_entries_scanned; /* adjacency entries read by the refine kernels               */
  int64_t repartitioned;   /* 1 iff the fallback policy (igk_options.fgp_fallback_ppm) ran a full
                              repartition at the end of this call; cut / max_part_weight are
                              then those of the new partition                                 */
} igk_refine_stats;

/* Create a handle from a symmetric CSR graph.  n vertices with IDs
 * 0..n-1; xadj[n+1] (int64), adjncy[xadj[n]] (no self loops, no duplicate
 * neighbours, symmetric), vwgt[n] in [1,65535] or NULL (unit), adjwgt
 * [xadj[n]] in [1,255] and symmetric, or NULL (unit); 2 <= k <= 254;
 * 0 < epsilon <= 1 (imbalance ratio); init_part[n] in [0,k) (need not
 * be balanced: the first igk_refine restores balance).  opt may be NULL.
 * Returns IGK_EINVAL (no handle) on invalid input. */
igk_status igk_create(const igk_options* opt, int64_t n, const int64_t* xadj,
                      const int32_t* adjncy, const int32_t* vwgt, const int32_t* adjwgt,
                      int32_t k, double epsilon, const int32_t* init_part, igk_graph** out);

/* Apply one batch of modifiers (S1, Alg. 1-2; Alg. 3 L1-7 marking).
 * The whole batch is validated on the device first; any invalid modifier ->
 * IGK_EINVAL, nothing changes, and *bad_index (nullable) = the lowest
 * invalid index.  Validity (against the pre-batch graph): no self loops; an
 * undirected edge appears at most once among the batch's edge modifiers;
 * EDGE_DELETE needs an existing edge whose endpoints are not deleted in the
 * batch; VERTEX_DELETE needs an active vertex, at most once; EDGE_INSERT
 * needs an absent edge whose endpoints are active and not deleted in the
 * batch, or inserted in this batch (the j-th VERTEX_INSERT gets ID
 * n_total + j); weights in range.  Phase order: edge deletions, vertex
 * deletions, vertex insertions, edge insertions; inside a phase the batch
 * order is irrelevant.  *first_new_id (nullable) = ID of the 1st insertion.
 * mods is a HOST array, copied before the call returns: a page-locked
 * buffer (cudaHostAlloc / cudaHostRegister / torch pin_memory) is DMA'd
 * straight to the device, pageable memory through an internal pinned
 * staging buffer. */
igk_status igk_apply_modifiers(igk_graph* g, const igk_modifier* mods, int64_t count,
                               int64_t* first_new_id, int64_t* bad_index);
/* Same, with mods in DEVICE memory (count entries on the handle's device). */
igk_status igk_apply_modifiers_device(igk_graph* g, const igk_modifier* d_mods, int64_t count,
                                      int64_t* first_new_id, int64_t* bad_index);

/* Incremental refinement (Sec. V.C; R1 filter, R2 expansion, R3 balance
 * restoration, R4 rounds of Alg. 4).  stats may be NULL.  Returns IGK_OK, or
 * IGK_WIMBALANCED in the weighted corner case (result still valid). */
igk_status igk_refine(igk_graph* g, igk_refine_stats* stats);

/* Global boundary refinement (G-kway "refines all
 * vertices on the partition boundary (i.e., vertices with adj_ext != 0)").
 * Every active placed vertex with a neighbour in another part -- or a pending
 * (pseudo) neighbour, which counts as external (reading Q13) -- joins the
 * affected set A on the partition as it stands when the call is made (reading
 * B1); then the ordinary refine (R1-R4) runs in the SAME kernel
 * launch.  A from earlier applies is kept (A |= boundary).  Intended to be
 * called periodically to undo the cut drift of many incremental iterations
 * (P:322).  Same arguments, stats and return codes as igk_refine;
 * stats->affected counts the boundary as affected. */
igk_status igk_refine_global(igk_graph* g, igk_refine_stats* stats);  /* one GPU only (EINVAL when sharded) */

/* One incremental iteration: igk_apply_modifiers + igk_refine fused (both
 * kernels launched back to back, one host synchronisation).  If the batch is
 * invalid, returns IGK_EINVAL exactly as igk_apply_modifiers would (nothing
 * changed; the refine was skipped) and *bad_index is set.  mods is a HOST
 * array (staged as in igk_apply_modifiers); igk_step_device takes a DEVICE array. */
igk_status igk_step(igk_graph* g, const igk_modifier* mods, int64_t count, igk_refine_stats* stats,
                    int64_t* first_new_id, int64_t* bad_index);
igk_status igk_step_device(igk_graph* g, const igk_modifier* d_mods, int64_t count, igk_refine_stats* stats,
                           int64_t* first_new_id, int64_t* bad_index);

/* Pipelined steps (store maintenance / IO): the next
 * batch's host->device copy overlaps the running step.
 *   igk_stage_batch  copies a HOST batch into one of two device buffers on
 *                    the handle's own copy stream and returns at once (a
 *                    page-locked buffer is DMA'd directly and must stay
 *                    unchanged until the igk_step_end of the step that
 *                    consumes it; pageable memory is copied into a pinned
 *                    staging buffer first).
 *   igk_step_begin   launches apply + refine on the most recently staged
 *                    batch (ordered after its copy) and returns without
 *                    waiting.
 *   igk_step_end     waits for that step; results, statuses and the
 *                    capacity retry exactly as igk_step.
 * Loop: stage(b0); for t: begin(); stage(b_t+1); end(); -- at most one step
 * in flight and one batch staged ahead.  Single-GPU handles only. */
igk_status igk_stage_batch(igk_graph* g, const igk_modifier* mods, int64_t count);
igk_status igk_step_begin(igk_graph* g);
igk_status igk_step_end(igk_graph* g, igk_refine_stats* stats, int64_t* first_new_id, int64_t* bad_index);

/* NEXT-2: full partitioning of a CSR graph on the GPU (IGK-FGP v1, DESIGN.md
 * 4 readings F1-F6): G-kway-style union-find coarsening with the paper's
 * constrained grouping (vertices of a subset sorted by their join
 * iteration and split into groups of group_size, the paper's s = 6), stop
 * below 35 k vertices or when fewer than 90% of the vertices could be
 * coarsened, a greedy initial partition of the coarsest graph, and at
 * every level the projection + global boundary refinement (igk_refine_global
 * on a wide-weight handle, repeated while it lowers the cut, <= 8 passes).
 * Inputs as igk_create (host CSR; weights up to INT32_MAX with totals <=
 * INT32_MAX); opt: device / stream (NULL = defaults).  part_out[n] gets the
 * partition; level_n (nullable, >= 33 entries) the vertices per level;
 * *nlevels (nullable) the number of levels.  IGK_EINVAL on invalid input;
 * the reason of a failure is in igk_last_error(NULL). */
igk_status igk_fgp_partition(const igk_options* opt, int64_t n, const int64_t* xadj, const int32_t* adjncy,
                             const int32_t* vwgt, const int32_t* adjwgt, int32_t k, double epsilon,
                             int32_t group_size, int32_t* part_out, int64_t* level_n, int32_t* nlevels);

/* NEXT-2: full repartition of a handle's current graph in place (
 * reading F8): the active vertices are relabelled densely in ID
 * order, their induced graph (rows ascending) goes through the same device
 * pipeline as igk_fgp_partition with the handle's k and epsilon, and the
 * parts are written back (deleted vertices stay deleted); the maintained cut
 * and W_p are recounted.  Everything runs on the device (no host copy of the
 * graph).  IGK_ESTATE if a batch was applied and not yet refined, or after
 * a CUDA error; IGK_EINVAL for sharded / wide handles or group_size < 2.
 * *out_cut (nullable) = the new cut.  Afterwards igk_partition_delta
 * returns IGK_ESTATE until the next refine (read igk_partition). */
igk_status igk_repartition(igk_graph* g, int32_t group_size, int64_t* out_cut);

/* NCCL unique id for sharded handles (call on ONE rank, share the 128
 * bytes with the others, pass as igk_options.nccl_id).  NCCL is loaded at
 * run time (libnccl.so.2); IGK_ENCCL if it is unavailable. */
igk_status igk_nccl_unique_id(void* out, int64_t len);

/* The k-way partition (V_1..V_k; P:50 the part of every vertex).
 * out[v] for v < n_total: part in [0,k), -1 = deleted, -2 = pending (in the
 * pseudo-partition between apply and refine).  out is a HOST buffer of
 * cap_len entries; cap_len too small -> IGK_EINVAL with *n_total still set
 * (call with out == NULL to query the size).  One device gather + one D2H. */
igk_status igk_partition(const igk_graph* g, int32_t* out, int64_t cap_len, int64_t* n_total);
/* The partition CHANGES of the last igk_refine / igk_refine_global /
 * igk_step: (vertex, new part) int32 pairs, one per vertex whose part now
 * differs from its part before that refine -- the frontier vertices that
 * moved (only they can, invariant I4) and every vertex inserted
 * since the previous refine (its first placement, Alg. 3 L2-5).  Vertices
 * deleted by the batch are not listed (the caller issued those deletions).
 * This is what an IGP-in-the-loop client consumes each iteration
 * instead of the whole vector.  pairs: HOST buffer of 2 * cap int32 (pair
 * order unspecified); *count = number of pairs.  cap < count -> IGK_EINVAL
 * with *count set (pairs == NULL queries the count).  The list is built on
 * the device by the refine kernel; this call is one D2H of 8 * count bytes
 * (page-locked `pairs` are DMA'd directly). */
igk_status igk_partition_delta(const igk_graph* g, int32_t* pairs, int64_t cap, int64_t* count);
/* cut size, maintained incrementally; edges with a pending endpoint
 * are not counted. */
igk_status igk_cut_size(const igk_graph* g, int64_t* out);
/* part weights W_p, k entries */
igk_status igk_part_weights(const igk_graph* g, int64_t* out_k);
/* |V| bookkeeping (P:48 V; vertex_status): *n_total = IDs in use
 * (deleted IDs are never reused), *n_active = active vertices (a device
 * reduction over the labels, one 8-byte read back).  Either may be NULL. */
igk_status igk_num_vertices(const igk_graph* g, int64_t* n_total, int64_t* n_active);
/* Recount cut and W_p from scratch with the cut/weight reduction kernel
 * (S9: cut = sum of W_e over edges whose endpoints lie in different parts,
 * W_p = sum of vertex weights per part; pending vertices count for no
 * part).  One cooperative launch of k_recount3 (HBM-bound full store scan,
 * DESIGN.md 6); the environment variable IGK_RECOUNT=gather|tma read at
 * igk_create selects the round-1 gather kernel or the TMA variant instead
 * (A/B only).  Synchronises the handle's stream.  out_cut: 1 value, out_wp:
 * k values (may be NULL), host memory owned by the caller.  Errors:
 * IGK_ESTATE on a poisoned handle, IGK_ECUDA if a CUDA call fails. */
igk_status igk_recount(igk_graph* g, int64_t* out_cut, int64_t* out_wp);
/* Debug/test: current graph as a symmetric CSR over all IDs (deleted rows
 * empty; order inside a row unspecified).  Size query: call with xadj ==
 * NULL to get *n_total and *n_slots.  Built on the device (live-degree scan
 * + row gather kernel) and read back in one copy per output array. */
igk_status igk_export_csr(const igk_graph* g, int64_t* xadj, int64_t xadj_len, int32_t* adjncy,
                          int32_t* adjwgt, int64_t adj_len, int64_t* n_total, int64_t* n_slots);
/* store occupancy: IDs in use, active vertices and live (directed)
 * adjacency entries (= 2m) as of the last igk_recount, slab bump pointer
 * and capacity (entries) */
igk_status igk_store_stats(const igk_graph* g, int64_t* n_total, int64_t* n_active, int64_t* adj_entries,
                           int64_t* slab_top, int64_t* slab_cap);
/* Store maintenance (NEXT-4): rewrite the adjacency slab densely (drops
 * tombstones and the holes relocations leave), growing it if needed.  Also
 * done automatically: when a batch fails validation only for capacity (vertex
 * IDs or slab slots; nothing is modified then), the library grows the vertex
 * arrays and/or compacts the slab and re-runs the batch once. */
igk_status igk_compact(igk_graph* g);
/* number of kernels this handle has launched so far (instrumentation) */
int64_t igk_kernel_launches(const igk_graph* g);
/* instrumentation: how often each rarely-taken code path ran since
 * igk_create, so tests can show every path the full-size inputs need was
 * exercised.  out[i] for i < returned count (<= cap), index = IGK_PATH_*. */
enum {
  IGK_PATH_HUB_FILTER = 0,  /* filter of a hub (degree > 1024) by a whole CTA           */
  IGK_PATH_HUB_COMMIT,      /* commit of a hub candidate by a whole CTA                 */
  IGK_PATH_HUB_GAIN,        /* round gain of a pending hub by a whole CTA               */
  IGK_PATH_TIE_CTA,         /* cutoff round: an overflowing part's tie group in one CTA */
  IGK_PATH_TIE_GRID,        /* cutoff round: grid-wide radix passes (fallback)          */
  IGK_PATH_KEY_EXACT,       /* cutoff threshold digit with #nbr < 255 (ID key)          */
  IGK_PATH_KEY64,           /* cutoff threshold digit with #nbr >= 255 (64-bit key)     */
  IGK_PATH_FORCED_L0,       /* L = 0: first sorted move forced (reading Q8)             */
  IGK_PATH_WFALLBACK,       /* E(u) empty: lightest part + imbalance flag (Q8)          */
  IGK_PATH_R3,              /* balance restoration ran                                   */
  IGK_PATH_R3_KEY64,        /* restoration threshold in a clamped loss digit             */
  IGK_PATH_RELOC,           /* prefixes relocated on overflow                            */
  IGK_PATH_VDEL_WARP,       /* vertex deletions, warp per 8-entry item                   */
  IGK_PATH_VDEL_THREAD,     /* vertex deletions, thread per 8-entry item                 */
  IGK_PATH_WARP_GAIN,       /* round gains in the warp bucket (degree 17..1024)          */
  IGK_PATH_RESERVED15,
  IGK_PATH_COMPACTION = 16, /* slab compactions (host)                                   */
  IGK_PATH_VERTEX_GROWTH,   /* vertex-array growths (host)                               */
  IGK_PATH_SPLIT_STEP,      /* igk_step as k_apply + k_refine (large batch)              */
  IGK_PATH_FUSED_STEP,      /* igk_step as one k_step                                    */
  IGK_PATH_NOTICE_FALLBACK, /* step completion notice missed: copy + sync fallback       */
  IGK_PATH_N
};
int32_t igk_debug_paths(const igk_graph* g, int64_t* out, int32_t cap);
/* instrumentation: profile mode on/off.  On: every refine records the
 * %globaltimer phase stamps (igk_debug_phase_times) and, per phase, the
 * adjacency entries scanned and the list items processed
 * (igk_debug_phase_work), for per-phase roofline accounting; the step's
 * fast completion notice is replaced by a full control-block copy. */
igk_status igk_debug_set_profile(igk_graph* g, int32_t on);
/* per-phase work of the last refine in profile mode, index = phase:
 * 0 boundary scan (igk_refine_global), 1 F0 R1 filter, 2 F1 commit C1 +
 * expansion marks, 3 F2 R2 filter, 4 F3 commit C2, 5 R3 restoration,
 * 6 round gain (all rounds), 7 round prefix select + move (all rounds).
 * Returns the number of phases written (<= cap). */
int32_t igk_debug_phase_work(const igk_graph* g, int64_t* scanned, int64_t* items, int32_t cap);
/* device-side duration (ms) of the last igk_refine / apply / recount kernel,
 * measured with CUDA events on the handle's stream */
igk_status igk_last_kernel_ms(const igk_graph* g, float* refine_ms, float* apply_ms, float* recount_ms);
/* instrumentation: %globaltimer stamps (ns, relative to the kernel start)
 * taken by CTA 0 after every grid barrier of the last apply (which = 0) or
 * refine (which = 1) kernel; ids name the phase (see csrc/*.cuh).  Returns
 * the number of stamps written (<= cap). */
int32_t igk_debug_phase_times(const igk_graph* g, int32_t which, int32_t* ids, int64_t* t_ns, int32_t cap);
/* instrumentation (only if the environment had IGK_DEBUG_ARRIVALS set at
 * igk_create): per-CTA %globaltimer arrival stamps at barrier slot s of the
 * last kernel, out[s * grid + cta], 128 slots; returns the grid size.
 * which = 2: per-warp diagnostics of the last F1 commit pass (out[0, 4096):
 * end times, out[4096, 8192): heaviest prefix handled, + 2^20 if it was a
 * commit on the warp path); returns the number of warps. */
int32_t igk_debug_arrivals(const igk_graph* g, int32_t which, int64_t* out, int32_t cap);
/* the last failure of g; with g == NULL: why this thread's last igk_create failed */
const char* igk_last_error(const igk_graph* g);
void igk_destroy(igk_graph* g);

#ifdef __cplusplus
}
#endif
#endif
