// common.cuh -- device state, constants and warp/block helpers for libigk.
//
// Product code (sm_100a).  Shares nothing with oracle/ (see DESIGN.md 5).
#pragma once
#include <cooperative_groups.h>
#include <cuda_runtime.h>
#include <stddef.h>
#include <stdint.h>

namespace igk {
namespace cg = cooperative_groups;

// ---------------------------------------------------------------------------
// limits and labels
// ---------------------------------------------------------------------------
constexpr int kMaxK = 254;
constexpr uint8_t kPsi = 255;  // pseudo-partition label
constexpr uint8_t kDel = 254;  // deleted vertex (vertex_status = deleted)
constexpr int kVwMax = 65535;
constexpr int kEwMax = 255;
constexpr int kDegMax = 1 << 23;
constexpr int64_t kNMax = int64_t(1) << 30;
#ifndef IGK_THREADS
#define IGK_THREADS 512
#endif
constexpr int kThreads = IGK_THREADS;  // persistent-kernel block size (A/B builds: -DIGK_THREADS=...)
constexpr int kWarps = kThreads / 32;
#ifndef IGK_THREADDEG
#define IGK_THREADDEG 8
#endif
constexpr int kThreadDeg = IGK_THREADDEG;  // degree <= this: one thread per vertex; above: one warp (A/B: -DIGK_THREADDEG)
#ifndef IGK_BLOCKDEG
#define IGK_BLOCKDEG 1024
#endif
constexpr int kBlockDeg = IGK_BLOCKDEG;  // degree > this (hubs): one whole CTA per vertex (A/B: -DIGK_BLOCKDEG)
constexpr int kVdC = 8;            // vertex deletion: prefix entries per work item (one thread each)
constexpr int kDigits = 256;        // radix digit bins (8-bit digits)
constexpr long long kNoErr = 0x7fffffffffffffffLL;

enum ModKind { kEdgeDel = 0, kVertDel = 1, kVertIns = 2, kEdgeIns = 3 };

// ---------------------------------------------------------------------------
// control block in device memory: scalars, counters, stats
// ---------------------------------------------------------------------------
enum StatIdx {
  ST_AFFECTED = 0, ST_INSERTED, ST_EXPANDED, ST_FILTERED_IN, ST_EXPANDED_IN, ST_EVICTED,
  ST_ROUNDS, ST_MOVES_APPLIED, ST_MOVES_DEFERRED, ST_CUT, ST_CAP, ST_MAXW, ST_IMBAL, ST_SCANNED,
  ST_N
};

// Device path counters (igk_debug_paths): how often each rarely-taken code
// path ran since igk_create -- so the tests can show that every path the
// full-size inputs need was exercised (and bit-exact).  Order = igk.h IGK_PATH_*.
enum PathIdx {
  PA_HUB_FILTER = 0,  // filter of a hub (degree > kBlockDeg) by a whole CTA
  PA_HUB_COMMIT,      // commit of a hub candidate by a whole CTA
  PA_HUB_GAIN,        // round gain of a pending hub by a whole CTA
  PA_TIE_CTA,         // cutoff round: an overflowing part's tie group finished in one CTA
  PA_TIE_GRID,        // cutoff round: grid-wide radix passes over the tie groups (fallback)
  PA_KEY_EXACT,       // cutoff round threshold in an exact-key digit (#nbr < 255): 32-bit ID key
  PA_KEY64,           // cutoff round threshold in digit 0 (#nbr >= 255): 64-bit (#nbr, ID) key
  PA_FORCED_L0,       // L = 0: the first sorted move forced (reading Q8)
  PA_WFALLBACK,       // E(u) empty: move to the lightest part with the imbalance flag (Q8)
  PA_R3,              // balance restoration ran (some W_p > cap)
  PA_R3_KEY64,        // restoration threshold in a clamped (non-exact) loss digit
  PA_RELOC,           // prefixes relocated on overflow (apply M3)
  PA_VDEL_WARP,       // vertex deletions: one warp per 8-entry item
  PA_VDEL_THREAD,     // vertex deletions: one thread per 8-entry item
  PA_WARP_GAIN,       // rounds that ran the warp bucket of the gain (degree 17..1024)
  PA_N_DEV = 16
};

struct Ctl {
  // ---- outputs read back after every call (kept first: lean D2H copy) ----
  long long n_total;   // vertex IDs in use
  long long slab_top;  // bump pointer of the adjacency slab
  long long W;         // total active vertex weight
  long long cut;       // maintained cut (placed endpoints only)
  long long err_idx;   // lowest invalid modifier index (kNoErr = none)
  long long st_out[ST_N];  // stats of the last refine (copied at its end)
  int err_nomem;
  int n_ins;
  int refine_skipped;  // fused step: refine skipped because the batch was rejected
  int nph;             // phase timestamps recorded by the last kernel
  int nrec;            // sharded round: move records emitted by this rank
  int rs_cur;          // sharded refine: round state between host-driven launches
  long long rs_rounds, rs_rounds_all, rs_applied, rs_deferred;
  int rs_pending;      // pending vertices left for the next sharded round
  long long slab_need; // slots the last rejected batch asked for (capacity failure: sizes the compaction)
  int n_delta;         // (vertex, part) pairs in the delta list of the last refine
  int sh_flag;         // sharded refine: restoration (R3) needed after kShF3
  int sh_np;           // sharded refine: pending vertices after F3 / R3 (length of the canonical list)
  int p2p_err;         // persistent P2P rounds: a peer never reached the device barrier (timeout)
  long long sh_err[2]; // sharded apply: [0] lowest invalid index, [1] capacity flags (all-reduced MIN / MAX)
  // ---- device-side state ----
  long long Wp[256];   // part weights
  long long tot3[3][256];  // per round (mod 3): weight of selected moves per target part
  long long slab_top0;     // slab_top before the current apply (rollback)
  long long st[ST_N];  // refine stats (accumulating)
  int nA;              // affected list length
  int nhubA, nhubC, nhubN, nhubC2, nhubP;  // hub (degree > kBlockDeg) work lists
  int npsi[3];         // pseudo list lengths
  int ncand;           // candidate list length (C1, R3)
  int ncand2;          // candidate list length (C2)
  int nN;              // expansion list length
  int ngrow;           // relocation list length
  int nreloc;          // relocation list length
  int nr3;             // restoration candidate list length
  int nvdch;           // vertex-deletion work chunks
  int ntie;            // tie-group buffer length (round prefix select)
  int tiecnt[256];     // tie-group size per part
  unsigned long long kres[256];  // per-part threshold keys from the CTA-local select
  int applied3[3];     // moves applied per round (mod 3)
  int selected3[3];    // moves selected per round (mod 3)
  unsigned long long tph[128];  // %globaltimer after each phase (CTA 0)
  int idph[128];                // phase ids
  int ndone;                    // CTAs finished (publish: the last one posts the notice)
  int ndone_ref;                // CTAs past the refine epilogue (the last one finalises the stats)
  long long paths[PA_N_DEV];    // device path counters (cumulative)
  long long phscan[8];          // profile mode: adjacency entries scanned per refine phase (PH_*)
  long long phitems[8];         // profile mode: list items (vertices) processed per refine phase
};
// refine phases of the per-phase work counters (igk_debug_phase_work)
enum PhaseIdx { PH_BOUNDARY = 0, PH_F0, PH_F1, PH_F2, PH_F3, PH_R3, PH_GAIN, PH_MOVE, PH_N };
__device__ __forceinline__ void path_hit(Ctl* ctl, int which, long long v = 1) {
  atomicAdd((unsigned long long*)&ctl->paths[which], (unsigned long long)v);
}

// ---------------------------------------------------------------------------
// all device pointers of one handle, passed by value to every kernel
// ---------------------------------------------------------------------------
// Per-vertex store record, 16 bytes = one aligned half-sector: the fields a
// vertex visit reads together (offset and length of its dense prefix) come
// in ONE memory transaction instead of one cold miss per array.
struct __align__(16) VRec {
  int64_t off;   // slab offset of the vertex's dense prefix (multiple of 4)
  int32_t deg;   // prefix length (live entries + tombstones, -1)
  int32_t ldeg;  // live degree (tombstones excluded)
};

struct Dev {
  int32_t k;
  int64_t n_cap;     // vertex capacity
  int64_t slot_cap;  // slab capacity (entries)
  int32_t slack_min;
  int32_t idbits;    // bits to hold any vertex ID < n_cap
  // vertex-range sharding: rank `rank` of `nranks` owns the IDs
  // [rank * sh_blk, (rank + 1) * sh_blk) of the created graph and the inserted
  // IDs n with (n - sh_n0) % nranks == rank.  It stores the adjacency of its
  // own vertices in full and, for every other vertex, the "ghost" prefix of
  // its neighbours that this rank owns, so both directions of every edge it
  // touches are local (twins stay valid).  nranks == 1: one GPU owns all.
  int32_t nranks, rank;
  int32_t sharded;   // the sharded protocol runs (nranks > 1, or a transport given for one rank)
  int64_t sh_n0, sh_blk;
  uint64_t* bm;      // sharded refine: candidate bitmap (n_cap bits), all-reduced (sum of disjoint bits = OR)
  uint32_t* lossbuf; // sharded R3: (int - ext) + 2^31 of owned restoration candidates, 0 = none; all-reduced
  int4* recs;        // sharded rounds: one move record per position of the canonical pending list
  // NEXT-3 persistent round kernel: the round's record buffer of every rank
  // (peer memory over NVLink P2P, or the same device); the gain stores each
  // record into all of them
  int32_t p2p_n;
  int4* p2p_recs[8];
  // graph store (S0)
  VRec* vr;          // per-vertex record: prefix offset, length, live degree (one sector)
  int32_t* capv;     // capacity
  int32_t* adj;      // neighbour IDs (-1 = tombstone)
  int32_t* twin;     // slot of the reverse entry (x -> u) of every live slot (u -> x)
  int32_t* adjw;     // edge weights (nullptr = unit)
  uint8_t* active;
  int32_t* vw;       // vertex weights (nullptr = unit)
  uint8_t* part;
  // stamps (epoch marks; never cleared)
  uint32_t* markA;   // membership in the affected set A
  uint32_t* markT;   // temporary sets (candidates, N, dirty)
  uint32_t* markD;   // deleted-in-batch
  uint32_t* markG;   // first touch by an edge insertion (grow list)
  int32_t* vcnt;     // VERTEX_DELETE count per vertex (zero between calls)
  int32_t* icnt;     // EDGE_INSERT count per endpoint (zero between calls)
  // lists (n_cap entries each)
  int32_t* Alist;
  int32_t* psi[3];    // [0] accumulates Psi (= frontier F); [1],[2] round buffers
  int32_t* cand;
  int32_t* cand2;
  int32_t* Nlist;
  int32_t* glist;    // grow / relocation list
  int32_t* rlist;    // relocation list: first-touched vertices whose prefix moves (V2)
  int2* r3list;      // (vertex, loss) restoration candidates
  int2* vdch;        // (vertex, chunk) work items of vertex deletions, kVdC entries each
  uint32_t* markF;   // frontier membership (entered Psi in this refine cycle)
  uint32_t* markH;   // hub routed to a CTA-cooperative list (epoch = the list's cycle)
  int32_t* hubA;     // hubs in A
  int32_t* hubC;     // hub candidates of R1 / R2 / R3 (commit lists)
  int32_t* hubN;     // hubs in N (R2)
  int32_t* hubC2;
  int32_t* hubP;     // hubs in the pseudo-partition (rounds)
  uint8_t* oldp;     // part before entering Psi (kPsi for inserted vertices)
  int64_t* reloc;    // new slab offset for relocated vertices
  // per-vertex move results (rounds)
  uint8_t* tgt;
  int32_t* gain;
  int32_t* pw;       // placed-neighbour weight at round start (cut delta of a placement)
  uint32_t* meta;    // per psi index: bit31 selected | d0 << 8 | p*
  uint32_t* metav;   // per vertex: the same record for CTA-processed hubs
  // selection histograms
  long long* hist0;  // [256][256] digit-0 weights per part
  long long* histR;  // [3][256][256] pass histograms
  // apply scratch
  unsigned long long* hkeys;  // dup-detection hash (keys)
  int32_t* hcnt;              // dup-detection hash (counts)
  int64_t hmask;
  int32_t* blkcnt;            // per-block counts for chunked scans
  int32_t* newid;             // per modifier: new vertex ID of a VERTEX_INSERT
  int2* delta;                // (vertex, new part) of every label change of the last refine
  unsigned long long* dbg;    // optional per-CTA barrier arrival stamps [128][grid]
  Ctl* ctl;
  Ctl* hmap;                  // host-mapped copy of the output head (igk_step fast path)
  volatile unsigned* hflag;   // host-mapped completion notice
  unsigned seq;               // notice value of this launch (0 = no notice)
};

// ---------------------------------------------------------------------------
// helpers
// ---------------------------------------------------------------------------
// the rank owning vertex v (its full adjacency lives there); any v on one GPU
__host__ __device__ __forceinline__ bool own(const Dev& d, long long v) {
  if (d.nranks <= 1) return true;
  if (v < 0) return false;
  const long long r = v < d.sh_n0 ? v / d.sh_blk : (v - d.sh_n0) % d.nranks;
  return r == d.rank;
}
__device__ __forceinline__ long long ldv(const long long* p) { return *(volatile const long long*)p; }
__device__ __forceinline__ int ldv(const int* p) { return *(volatile const int*)p; }
__device__ __forceinline__ uint8_t ld_part(const uint8_t* p, int64_t i) { return __ldcg(p + i); }
// Loads of the store (adjacency, weights, vertex records) in the apply /
// refine kernels.  The fused k_step writes that data in its apply half and
// reads it in its refine half, so the non-coherent read-only path (__ldg,
// ld.global.nc: data must not change during the kernel) is never used for
// it: every such load goes through L2 (ld.global.cg).
template <typename T>
__device__ __forceinline__ T ldro(const T* p) {
  return __ldcg(p);
}

// one 16-byte load of a vertex record's (offset, prefix length) through L2
// (written in-kernel by the apply half of k_step, see ldro)
__device__ __forceinline__ void vr_ld(const Dev& d, int64_t u, long long& o, int& dg) {
  const longlong2 r = __ldcg(reinterpret_cast<const longlong2*>(d.vr + u));
  o = r.x;
  dg = (int)(unsigned)(unsigned long long)r.y;
}
__device__ __forceinline__ void vr_ldcg(const Dev& d, int64_t u, long long& o, int& dg) {
  const longlong2 r = __ldcg(reinterpret_cast<const longlong2*>(d.vr + u));
  o = r.x;
  dg = (int)(unsigned)(unsigned long long)r.y;
}

__device__ __forceinline__ int lane_id() { return threadIdx.x & 31; }
__device__ __forceinline__ int warp_id() { return threadIdx.x >> 5; }

__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}
// Completion notice for the host (igk_step fast path): the last CTA to
// finish copies the output head of Ctl into host-mapped memory, fences at
// system scope and raises the flag to this launch's sequence number.  The
// host polls the flag instead of a D2H copy + stream synchronisation.  Every
// CTA of the grid must call it exactly once, at its exit.
// the copy + flag half of publish(), for a CTA already known to be the last
__device__ __forceinline__ void publish_copy(const Dev& d);
__device__ __forceinline__ void publish(const Dev& d) {
  if (d.seq == 0) return;
  __shared__ int s_last;
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    s_last = atomicAdd(&d.ctl->ndone, 1) == (int)gridDim.x - 1;
  }
  __syncthreads();
  if (!s_last) return;
  publish_copy(d);
}
__device__ __forceinline__ void publish_copy(const Dev& d) {
  if (d.seq == 0) return;
  __threadfence();
  const int nw = (int)(offsetof(Ctl, Wp) / 8);
  const long long* src = reinterpret_cast<const long long*>(d.ctl);
  long long* dst = reinterpret_cast<long long*>(d.hmap);
  for (int i = threadIdx.x; i < nw; i += blockDim.x) dst[i] = __ldcg(src + i);
  __threadfence_system();
  __syncthreads();
  if (threadIdx.x == 0) {
    d.ctl->ndone = 0;
    *d.hflag = d.seq;
    __threadfence_system();
  }
}

// phase stamp: CTA 0 / thread 0 records (id, time) right after a grid barrier
__device__ __forceinline__ void stamp_phase(Ctl* ctl, int id) {
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    int i = ctl->nph;
    if (i < 128) {
      ctl->tph[i] = gtimer();
      ctl->idph[i] = id;
      ctl->nph = i + 1;
    }
  }
}

// per-warp diagnostics region of the arrival buffer (past every slot row of
// grids up to 2048 CTAs): [kDbgWarp, +4096) times, [+4096, +8192) values
constexpr long long kDbgWarp = 64ll * 4096;
// opt-in instrumentation: every CTA stamps its arrival at barrier `slot`
__device__ __forceinline__ void arrive_stamp(unsigned long long* dbg, int slot) {
  if (dbg && slot < 128) {
    __syncthreads();
    if (threadIdx.x == 0) dbg[(long long)slot * gridDim.x + blockIdx.x] = gtimer();
  }
}

// grid barrier with instrumentation (CTA arrival stamp + CTA-0 phase stamp)
#define GRID_SYNC_STAMPED(ctl_, id_)      \
  do {                                    \
    arrive_stamp(d.dbg, (id_) % 100);     \
    grid.sync();                          \
    stamp_phase(ctl_, id_);               \
  } while (0)

// Flat loop over [0, n) in 32-item chunks (one chunk per warp, lanes
// contiguous so warp-aggregated appends stay one atomic per warp), with the
// chunks dealt CTA-first: chunk c -> CTA c mod G, warp (c / G) mod W.  A
// short list thus spreads over all SMs instead of filling the first CTAs.
template <class F>
__device__ __forceinline__ void rr_for(long long n, F f) {
  const long long G = gridDim.x, W = blockDim.x >> 5;
  const long long my = (long long)(threadIdx.x >> 5) * G + blockIdx.x;  // this warp's rank
  const long long nw = G * W;
  const long long nch = (n + 31) >> 5;
  for (long long c = my; c < nch; c += nw) {
    long long i = (c << 5) + (threadIdx.x & 31);
    if (i < n) f(i);
  }
}

// Warp-uniform variant of rr_for: f(i, valid) runs on every lane of the warp
// in every iteration (valid == false past the end), so f may use warp
// collectives (ballot loops for heavy items).
template <class F>
__device__ __forceinline__ void rr_for_warp(long long n, F f) {
  const long long G = gridDim.x, W = blockDim.x >> 5;
  const long long my = (long long)(threadIdx.x >> 5) * G + blockIdx.x;
  const long long nw = G * W;
  const long long nch = (n + 31) >> 5;
  for (long long c = my; c < nch; c += nw) {
    long long i = (c << 5) + (threadIdx.x & 31);
    f(i, i < n);
  }
}

// per-part accumulation in shared memory with lanes of equal key combined
// first (one shared atomic per distinct key per warp)
__device__ __forceinline__ void acc_add(long long* acc, int key, long long v) {
  unsigned act = __activemask();
  unsigned grp = __match_any_sync(act, key);
  int leader = __ffs(grp) - 1;
  // sum v over the group (lanes of grp) via shuffles from the leader's view
  long long sum = 0;
  for (unsigned m = grp; m; m &= m - 1) sum += __shfl_sync(grp, v, __ffs(m) - 1);
  if ((int)(threadIdx.x & 31) == leader) atomicAdd((unsigned long long*)&acc[key], (unsigned long long)sum);
}

// warp-aggregated append: returns the slot of this lane (or -1 if !pred)
__device__ __forceinline__ int agg_append(int* ctr, bool pred) {
  unsigned act = __activemask();
  unsigned m = __ballot_sync(act, pred);
  int lane = lane_id();
  int leader = __ffs(act) - 1;
  int base = 0;
  if (lane == leader && m) base = atomicAdd(ctr, __popc(m));
  base = __shfl_sync(act, base, leader);
  return pred ? base + __popc(m & ((1u << lane) - 1u)) : -1;
}

// warp-aggregated bump allocation: the converged lanes' amounts v (0 =
// none) are summed, ONE atomicAdd reserves the total, each lane gets its
// exclusive offset.  Replaces per-lane atomics on one hot counter.
template <typename T>
__device__ __forceinline__ T agg_alloc(T* ctr, T v) {
  const unsigned act = __activemask();
  const int lane = lane_id();
  T total = 0, excl = 0;
  for (unsigned m = act; m; m &= m - 1) {
    const int src = __ffs(m) - 1;
    const T vv = __shfl_sync(act, v, src);
    if (src < lane) excl += vv;
    total += vv;
  }
  const int leader = __ffs(act) - 1;
  T base = 0;
  if (lane == leader && total) base = atomicAdd(ctr, total);
  base = __shfl_sync(act, base, leader);
  return base + excl;
}

// three warp-aggregated bump allocations in ONE round of leader atomics (the
// three counters are independent, so their round trips overlap): per lane
// amounts (g, s, r) -> this lane's exclusive bases (bg, bs, br)
__device__ __forceinline__ void agg_alloc3(int* cg, int g, unsigned long long* cs, unsigned long long s, int* cr,
                                           int r, int& bg, unsigned long long& bs, int& br) {
  const unsigned act = __activemask();
  const int lane = lane_id();
  int tg = 0, eg = 0, tr = 0, er = 0;
  unsigned long long ts = 0, es = 0;
  for (unsigned m = act; m; m &= m - 1) {
    const int src = __ffs(m) - 1;
    const int vg = __shfl_sync(act, g, src);
    const unsigned long long vs = __shfl_sync(act, s, src);
    const int vr = __shfl_sync(act, r, src);
    if (src < lane) {
      eg += vg;
      es += vs;
      er += vr;
    }
    tg += vg;
    ts += vs;
    tr += vr;
  }
  const int leader = __ffs(act) - 1;
  int b1 = 0, b3 = 0;
  unsigned long long b2 = 0;
  if (lane == leader) {
    if (tg) b1 = atomicAdd(cg, tg);
    if (ts) b2 = atomicAdd(cs, ts);
    if (tr) b3 = atomicAdd(cr, tr);
  }
  bg = __shfl_sync(act, b1, leader) + eg;
  bs = __shfl_sync(act, b2, leader) + es;
  br = __shfl_sync(act, b3, leader) + er;
}

template <typename T>
__device__ __forceinline__ T warp_sum(T v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}

// block-wide sum of a 64-bit value, then one atomicAdd by thread 0
__device__ __forceinline__ void block_atomic_add(long long* dst, long long v, long long* sbuf) {
  v = warp_sum(v);
  if (lane_id() == 0) sbuf[warp_id()] = v;
  __syncthreads();
  if (threadIdx.x == 0) {
    long long s = 0;
    for (int w = 0; w < (int)(blockDim.x >> 5); w++) s += sbuf[w];
    if (s) atomicAdd((unsigned long long*)dst, (unsigned long long)s);
  }
  __syncthreads();
}

__device__ __forceinline__ void atomic_add_ll(long long* p, long long v) {
  atomicAdd((unsigned long long*)p, (unsigned long long)v);
}

// stamp-based set insertion: true iff this call added v to the set
__device__ __forceinline__ bool stamp_insert(uint32_t* mark, int64_t v, uint32_t epoch) {
  if (__ldcg(mark + v) == epoch) return false;
  return atomicExch(mark + v, epoch) != epoch;
}

__device__ __forceinline__ int edge_w(const int32_t* adjw, int64_t j) { return adjw ? ldro(adjw + j) : 1; }
__device__ __forceinline__ int vert_w(const int32_t* vw, int64_t v) { return vw ? ldro(vw + v) : 1; }

// cap(W) = max(floor(W (1e6 + e) / (1e6 k)), ceil(W / k))  (reading Q4)
__host__ __device__ __forceinline__ long long cap_of(long long W, long long e_ppm, int k) {
  unsigned __int128 num = (unsigned __int128)(unsigned long long)W * (unsigned long long)(1000000 + e_ppm);
  unsigned long long den = 1000000ull * (unsigned long long)k;
  long long a = (long long)(num / den);
  long long b = (W + k - 1) / k;
  return a > b ? a : b;
}

}  // namespace igk
