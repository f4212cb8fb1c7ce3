// refine.cuh -- incremental refinement (Sec. V.C) as one persistent kernel.
//
//   F0  R1 filter over the affected set A            (Alg. 3 L8-24)
//   F1  deferred commit of C1 to the pseudo-partition (Alg. 3 L25-26),
//       fused with the R2 expansion marks (neighbours of pseudo vertices)
//   F2  R2 filter on sigma2 | F3 commit of C2
//   R3  balance restoration (paper silent; reading Q9): evict the minimum-loss
//       vertices of every overweight part via a weighted device radix select
//   R4  rounds (Alg. 4) until the pseudo-partition is empty:
//       gain = selection (no smaller-ID pseudo neighbour) + best part in one
//       adjacency pass, O(deg + k) | balanced prefix = weighted radix select of
//       the first violating move in (#nbr desc, ID asc) order | apply
// The cut is kept exact inside the same phases: a commit subtracts the cut
// edges of its candidates (read on the snapshot via candidate stamps + saved
// labels, edges between two candidates once), a placement adds its placed-
// neighbour weight minus its gain (the selected set is independent).
// The paper's sort + k x M segmented scan is replaced by a select
// that yields the same prefix without sorting.
#pragma once
#include "common.cuh"
#include "apply.cuh"  // mark_affected (A membership), shared with the apply

namespace igk {

struct RefineArgs {
  long long e_ppm;
  uint32_t epC1, epN, epC2, epF, epE;
  uint32_t epA;     // stamp of the affected set (hubs in A carry markH == epA)
  int after_apply;  // fused step: skip (leave the state untouched) if the batch was rejected
  int global;       // NEXT-1: the partition boundary joins A before F0 (igk_refine_global)
  int prof;         // profile mode: per-phase work counters (Ctl::phscan / phitems)
};

// profile mode: the adjacency entries this thread scanned since the last
// flush go to the phase's counter (block reduction + one atomic per CTA)
struct PhaseWork {
  long long mark = 0;
};
#define PHASE_FLUSH(ph, items)                                                 \
  do {                                                                         \
    if (a.prof) {                                                              \
      block_atomic_add(&d.ctl->phscan[ph], scanned - pw_.mark, s.red);         \
      pw_.mark = scanned;                                                      \
      if (blockIdx.x == 0 && threadIdx.x == 0 && (items))                      \
        atomic_add_ll(&d.ctl->phitems[ph], (long long)(items));                \
    }                                                                          \
  } while (0)

// Sharded refine: vertex-range owners (common.cuh own()) hold
// the full adjacency of their vertices plus ghost prefixes; labels, weights,
// W_p are replicated.  The refine runs as a sequence of launches with one
// all-reduce between them (igk.cu refine_sharded):
//   kShF0     R1 filter of the OWNED affected vertices -> C1 bitmap
//   [all-reduce C1 bitmap]
//   kShF1     every rank lists C1 from the bitmap, commits it (W_p, labels:
//             replicated; cut delta: by the owner), marks the OWNED placed
//             neighbours of pseudo vertices (N), R2-filters them -> C2 bitmap
//   [all-reduce C2 bitmap]
//   kShF3     lists + commits C2; if a part is overweight, the owners write
//             the (int - ext) key of their vertices of overweight parts
//   [all-reduce keys]  kShR3  the replicated weighted select + eviction commit
//   [the pending list is sorted by ID: one canonical order on every rank]
//   per round: kShGain  owners of selected pending vertices write their move
//             record at the vertex's position of the canonical list
//   [all-reduce records]  kShFinish  every rank installs all records, takes
//             the same balanced prefix and applies it
//   kShPost   epilogue (stats, delta list)
// Every all-reduce is a SUM of disjoint contributions (each vertex has one
// owner), i.e. a fixed-size OR / gather -- no size exchange is needed.
enum RefineMode { kModeFull = 0, kShF0, kShF1, kShF3, kShR3, kShGain, kShFinish, kShPost };
struct ShardArgs {
  int mode;       // RefineMode
  long long np;   // kShGain / kShFinish: length of the canonical pending list (d.psi[1])
};

// ---------------------------------------------------------------------------
// neighbour iteration with several loads in flight
// ---------------------------------------------------------------------------
// thread: f(x, w, q) for each neighbour; a chunk issues all its ID/weight
// loads, then all its label loads, before f runs; f returns false to stop
#ifndef IGK_WARPU
#define IGK_WARPU 8
#endif
constexpr int kWU = IGK_WARPU;  // warp bucket: entries per lane per round trip (A/B: -DIGK_WARPU)
constexpr int kWB = 32 * kWU;   // entries per warp per round trip
constexpr int kTC = kThreadDeg;  // thread chunk (one round trip per thread-bucket vertex)
// the commit's thread chunk: five values per slot (ID, weight, label, stamp,
// saved label) plus the expansion marks -- 8 slots keep it off the local stack
constexpr int kTCc = 8;
template <class F>
__device__ __forceinline__ void nbrs_thread(const Dev& d, long long o, int dg, F f) {
  for (int i = 0; i < dg; i += kTC) {
    int x[kTC], w[kTC];
    uint8_t q[kTC];
#pragma unroll
    for (int t = 0; t < kTC; t++) {
      x[t] = (i + t < dg) ? ldro(d.adj + o + i + t) : -1;
      w[t] = (i + t < dg && d.adjw) ? ldro(d.adjw + o + i + t) : 1;
    }
#pragma unroll
    for (int t = 0; t < kTC; t++) q[t] = x[t] >= 0 ? ld_part(d.part, x[t]) : (uint8_t)0;
#pragma unroll
    for (int t = 0; t < kTC; t++)
      if (x[t] >= 0 && !f(x[t], w[t], q[t])) return;
  }
}

// R2 expansion marks for the neighbours of u: the placed ones join N once
// (stamp epN).  All stamp probes / exchanges of a chunk are in flight
// together and N is appended with one atomic per lane and chunk.
// mk0 / dg0: the neighbours' stamps and prefix lengths when the caller
// already loaded them in its own gather round trip (the commit), else null
template <int C>
__device__ __forceinline__ void mark_chunk(const Dev& d, const int* x, const uint8_t* q, uint32_t epN,
                                           uint32_t epC, const unsigned* mk0 = nullptr, const int* dg0 = nullptr) {
  bool want[C];
  int dgx[C];
#pragma unroll
  for (int t = 0; t < C; t++) {
    unsigned mk = mk0 ? mk0[t] : (x[t] >= 0 ? __ldcg(d.markT + x[t]) : epN);
    dgx[t] = dg0 ? dg0[t] : (x[t] >= 0 ? ldro(&d.vr[x[t]].deg) : 0);
    // C1 members are pseudo on sigma2; sharded: each rank lists its own vertices
    want[t] = x[t] >= 0 && q[t] != kPsi && mk != epN && mk != epC && own(d, x[t]);
  }
  unsigned old[C];
#pragma unroll
  for (int t = 0; t < C; t++) old[t] = want[t] ? atomicExch(d.markT + x[t], epN) : epN;
  int c = 0, ch = 0;
#pragma unroll
  for (int t = 0; t < C; t++) {
    c += old[t] != epN && dgx[t] <= kBlockDeg;
    ch += old[t] != epN && dgx[t] > kBlockDeg;
  }
  int slot = c ? atomicAdd(&d.ctl->nN, c) : 0;  // one reservation per lane and chunk
  int hslot = ch ? atomicAdd(&d.ctl->nhubN, ch) : 0;
#pragma unroll
  for (int t = 0; t < C; t++) {
    if (old[t] == epN) continue;
    if (dgx[t] > kBlockDeg) d.hubN[hslot++] = x[t];  // hubs are filtered by a whole CTA
    else d.Nlist[slot++] = x[t];
  }
}
__device__ __forceinline__ void mark_nbrs_thread(const Dev& d, long long o, int dg, uint32_t epN, uint32_t epC) {
  for (int i = 0; i < dg; i += kTC) {
    int x[kTC];
    uint8_t q[kTC];
#pragma unroll
    for (int t = 0; t < kTC; t++) x[t] = (i + t < dg) ? ldro(d.adj + o + i + t) : -1;
#pragma unroll
    for (int t = 0; t < kTC; t++) q[t] = x[t] >= 0 ? ld_part(d.part, x[t]) : (uint8_t)0;
    mark_chunk<kTC>(d, x, q, epN, epC);
  }
}
__device__ __forceinline__ void mark_nbrs_warp(const Dev& d, long long o, int dg, uint32_t epN, uint32_t epC) {
  for (int b = 0; b < dg; b += kWB) {
    int x[kWU];
    uint8_t q[kWU];
#pragma unroll
    for (int t = 0; t < kWU; t++) {
      int i = b + t * 32 + lane_id();
      x[t] = i < dg ? ldro(d.adj + o + i) : -1;
    }
#pragma unroll
    for (int t = 0; t < kWU; t++) q[t] = x[t] >= 0 ? ld_part(d.part, x[t]) : (uint8_t)0;
    mark_chunk<kWU>(d, x, q, epN, epC);
  }
}
// warp: lane-strided, 8 entries per lane per round trip (256 per warp)
template <class F>
__device__ __forceinline__ void nbrs_warp(const Dev& d, long long o, int dg, F f) {
  for (int b = 0; b < dg; b += kWB) {
    int x[kWU], w[kWU];
    uint8_t q[kWU];
#pragma unroll
    for (int t = 0; t < kWU; t++) {
      int i = b + t * 32 + lane_id();
      x[t] = i < dg ? ldro(d.adj + o + i) : -1;
      w[t] = (i < dg && d.adjw) ? ldro(d.adjw + o + i) : 1;
    }
#pragma unroll
    for (int t = 0; t < kWU; t++) q[t] = x[t] >= 0 ? ld_part(d.part, x[t]) : (uint8_t)0;
#pragma unroll
    for (int t = 0; t < kWU; t++)
      if (x[t] >= 0) f(x[t], w[t], q[t]);
  }
}

// nbrs_warp with an early exit after each 256-entry chunk once any lane's
// stop() holds (the round gain of a blocked vertex)
template <class F, class S>
__device__ __forceinline__ void nbrs_warp_until(const Dev& d, long long o, int dg, F f, S stop) {
  for (int b = 0; b < dg; b += kWB) {
    int x[kWU], w[kWU];
    uint8_t q[kWU];
#pragma unroll
    for (int t = 0; t < kWU; t++) {
      int i = b + t * 32 + lane_id();
      x[t] = i < dg ? ldro(d.adj + o + i) : -1;
      w[t] = (i < dg && d.adjw) ? ldro(d.adjw + o + i) : 1;
    }
#pragma unroll
    for (int t = 0; t < kWU; t++) q[t] = x[t] >= 0 ? ld_part(d.part, x[t]) : (uint8_t)0;
#pragma unroll
    for (int t = 0; t < kWU; t++)
      if (x[t] >= 0) f(x[t], w[t], q[t]);
    if (__any_sync(0xffffffffu, stop())) return;
  }
}

// Iterate a vertex list: degree <= kThreadDeg -> one thread, else the whole
// warp cooperates on it.  Items are dealt round-robin over ALL warps of the
// grid (item i -> warp i mod W, lane (i / W) mod 32), so a short list still
// spreads over every SM and heavy vertices rarely share a warp.
// get(i) -> list entry (vertex or -1); pre(u, i) -> the per-vertex word the
// bucket needs (its label, saved label, ...) or -1 to skip the vertex;
// tf(u, i, off, deg, pv) / wf(u, i, off, deg, pv).  The vertex record and
// pre's loads do not depend on each other, so they are issued together: one
// dependent round trip per item before the adjacency loads.
template <class Get, class Pre, class TF, class WF>
__device__ __forceinline__ void foreach_vertex(const Dev& d, long long n, Get get, Pre pre, TF tf, WF wf) {
  const long long nw = ((long long)gridDim.x * blockDim.x) >> 5;
  const long long gw = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const long long per_round = nw * 32;
  // (packing a short list into the lanes of one warp per CTA -- item
  // r0 + cta + G (lane + 32 warp), warp-aggregated appends -- measured
  // slower: C2 0.201 vs 0.185 ms per step, profiles/r02_z_*)
  auto item = [&](int ln) -> long long { return (long long)ln * nw + gw; };
  for (long long r0 = 0; r0 < n; r0 += per_round) {
    long long i = r0 + item(lane_id());
    int u = i < n ? get(i) : -1;
    long long o = 0;
    int dg = 0, pv = -1;
    if (u >= 0) {
      vr_ld(d, u, o, dg);  // one 16-byte record load; handed to the bucket
      pv = pre(u, i);
    }
    const bool ok = pv >= 0;
    const bool heavy = ok && dg > kThreadDeg;
    if (ok && !heavy) tf(u, i, o, dg, pv);
    unsigned hm = __ballot_sync(0xffffffffu, heavy);
    while (hm) {
      int src = __ffs(hm) - 1;
      hm &= hm - 1;
      int uu = __shfl_sync(0xffffffffu, u, src);
      long long oo = __shfl_sync(0xffffffffu, o, src);
      int dd = __shfl_sync(0xffffffffu, dg, src);
      int pp = __shfl_sync(0xffffffffu, pv, src);
      wf(uu, r0 + item(src), oo, dd, pp);
    }
  }
}

// ---------------------------------------------------------------------------
// weighted radix select (shared by R3 and the round prefix)
// Per candidate part p: find the first item, in ascending key order among the
// items of part p, whose inclusive weight prefix reaches T_p.  Key = (d0, R):
// d0 is an 8-bit digit histogrammed by the producing phase (d.hist0); R is the
// item's vertex ID when bin d0 is exact, else a full 64-bit key.  MSD passes
// of 8 bits over R, one grid barrier per pass; every CTA recomputes the digit
// choice from the global histograms, so the choice needs no extra barrier.
// ---------------------------------------------------------------------------
struct SelSmem {
  long long T[256];
  long long base[256];
  unsigned long long prefix[256];
  int shift[256];
  short d0[256];
  uint8_t exact[256];
  uint8_t active[256];
  uint8_t found[256];
  uint8_t used[256];
  int nactive;
};

// first digit d with h[d] > 0 and base + sum_{<=d} h >= T (warp-wide)
__device__ __forceinline__ bool warp_pick_digit(const long long* h, long long base, long long T, int& dsel,
                                                long long& before) {
  const int l = lane_id();
  long long v[8];
  long long s = 0;
#pragma unroll
  for (int t = 0; t < 8; t++) {
    v[t] = __ldcg(h + 8 * l + t);
    s += v[t];
  }
  long long incl = s;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    long long y = __shfl_up_sync(0xffffffffu, incl, o);
    if (l >= o) incl += y;
  }
  long long run = base + incl - s;
  int cd = -1;
  long long cb = 0;
#pragma unroll
  for (int t = 0; t < 8; t++) {
    if (cd < 0 && v[t] > 0) {
      if (run + v[t] >= T) {
        cd = 8 * l + t;
        cb = run;
      }
      run += v[t];
    }
  }
  unsigned m = __ballot_sync(0xffffffffu, cd >= 0);
  if (!m) return false;
  int src = __ffs(m) - 1;
  dsel = __shfl_sync(0xffffffffu, cd, src);
  before = __shfl_sync(0xffffffffu, cb, src);
  return true;
}

__device__ __forceinline__ bool key_less(int da, unsigned long long ra, int db, unsigned long long rb) {
  return da < db || (da == db && ra < rb);
}

template <class ExactFn>
__device__ void sel_digit0(const Dev& d, SelSmem& sm, ExactFn is_exact, int exact_shift) {
  for (int p = threadIdx.x; p < 256; p += blockDim.x) {
    sm.found[p] = 0;
    sm.active[p] = 0;
  }
  __syncthreads();
  for (int p = warp_id(); p < d.k; p += kWarps) {
    if (!sm.used[p]) continue;
    int dd;
    long long before;
    bool f = warp_pick_digit(d.hist0 + (long long)p * kDigits, 0, sm.T[p], dd, before);
    if (lane_id() == 0) {
      sm.found[p] = f;
      sm.active[p] = f;
      if (f) {
        sm.d0[p] = (short)dd;
        sm.base[p] = before;
        sm.exact[p] = is_exact(dd);
        sm.shift[p] = sm.exact[p] ? exact_shift : 56;
        sm.prefix[p] = 0;
      }
    }
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    int c = 0;
    for (int p = 0; p < d.k; p++) c += sm.active[p];
    sm.nactive = c;
  }
  __syncthreads();
}

template <class Items>
__device__ void sel_accumulate(const Dev& d, SelSmem& sm, int pass, long long nitems, Items items) {
  long long* hb = d.histR + (long long)(pass % 3) * 256 * kDigits;
  long long* hz = d.histR + (long long)((pass + 1) % 3) * 256 * kDigits;
  rr_for((long long)d.k * kDigits, [&](long long t) {
    if (sm.active[t / kDigits]) hz[t] = 0;
  });
  rr_for(nitems, [&](long long j) {
    int p, d0;
    unsigned long long R;
    long long w;
    if (!items(j, p, d0, R, w)) return;
    if (!sm.active[p] || d0 != sm.d0[p]) return;
    int sh = sm.shift[p];
    if (sh + 8 < 64 && (R >> (sh + 8)) != (sm.prefix[p] >> (sh + 8))) return;
    int dig = (int)((R >> sh) & 255);
    atomic_add_ll(hb + (long long)p * kDigits + dig, w);
  });
}

__device__ void sel_choose(const Dev& d, SelSmem& sm, int pass) {
  const long long* hb = d.histR + (long long)(pass % 3) * 256 * kDigits;
  for (int p = warp_id(); p < d.k; p += kWarps) {
    if (!sm.active[p]) continue;
    int dd;
    long long before;
    bool f = warp_pick_digit(hb + (long long)p * kDigits, sm.base[p], sm.T[p], dd, before);
    if (lane_id() == 0) {
      if (f) {  // always true: the threshold item lies inside the prefix range
        sm.prefix[p] |= (unsigned long long)dd << sm.shift[p];
        sm.base[p] = before;
      }
      sm.shift[p] -= 8;
      if (sm.shift[p] < 0) sm.active[p] = 0;
    }
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    int c = 0;
    for (int p = 0; p < d.k; p++) c += sm.active[p];
    sm.nactive = c;
  }
  __syncthreads();
}

template <class Items>
__device__ void sel_passes(const Dev& d, SelSmem& sm, cg::grid_group& grid, long long nitems, Items items) {
  int pass = 0;
  while (sm.nactive > 0) {
    sel_accumulate(d, sm, pass, nitems, items);
    arrive_stamp(d.dbg, 300 + pass - 200);
    grid.sync();
    stamp_phase(d.ctl, 300 + pass);
    sel_choose(d, sm, pass);
    pass++;
  }
  if (pass > 0) grid.sync();  // every CTA finished reading before anyone clears
}

template <class ExactFn, class Items>
__device__ void weighted_select(const Dev& d, SelSmem& sm, cg::grid_group& grid, ExactFn is_exact,
                                int exact_shift, long long nitems, Items items) {
  sel_digit0(d, sm, is_exact, exact_shift);
  sel_passes(d, sm, grid, nitems, items);
}

__device__ void sel_clear(const Dev& d, const SelSmem& sm) {
  rr_for((long long)d.k * kDigits, [&](long long t) {
    if (!sm.used[t / kDigits]) return;
    d.hist0[t] = 0;
    d.histR[t] = 0;
    d.histR[256 * kDigits + t] = 0;
    d.histR[2 * 256 * kDigits + t] = 0;
  });
}

// ---------------------------------------------------------------------------
// the refine kernel
// ---------------------------------------------------------------------------
constexpr int kTieMax = 4096;
constexpr unsigned kMetaHub = 0x40000000u;  // move record kept per vertex (metav): CTA-processed hub  // tie groups up to this size finish in one CTA's shared memory
struct RefSmem {
  SelSmem sel;
  int tie_u[kTieMax];     // CTA-local select: vertex IDs of one part's tie group
  int tie_w[kTieMax];     //                   and their weights
  long long tie_h[256];
  unsigned long long tie_prefix;
  long long tie_base;
  int tie_n;
  long long Wr[256];      // round-start part weights (Q14)
  long long acc[256];     // per-part weight deltas of this CTA
  long long red[2 * kWarps];
  int wconn[kWarps][256]; // per-warp connectivity histogram
  int best0;
};

__device__ __forceinline__ void flush_acc(RefSmem& s, long long* dst, int k) {
  __syncthreads();
  for (int p = threadIdx.x; p < k; p += blockDim.x) {
    if (s.acc[p]) atomic_add_ll(dst + p, s.acc[p]);
    s.acc[p] = 0;
  }
  __syncthreads();
}

// CTA-local weighted select over one part's tie group (vertex IDs < 2^31):
// the first ID, ascending, whose inclusive weight prefix (after `base`)
// reaches T.  Four 8-bit MSD passes over a shared-memory histogram.
__device__ unsigned block_select_ids(RefSmem& s, int cnt, long long base, long long T) {
  if (threadIdx.x == 0) {
    s.tie_prefix = 0;
    s.tie_base = base;
  }
  for (int shift = 24; shift >= 0; shift -= 8) {
    for (int b = threadIdx.x; b < 256; b += blockDim.x) s.tie_h[b] = 0;
    __syncthreads();
    const unsigned pre = (unsigned)s.tie_prefix;
    for (int i = threadIdx.x; i < cnt; i += blockDim.x) {
      unsigned u = (unsigned)s.tie_u[i];
      if (shift == 24 || (u >> (shift + 8)) == (pre >> (shift + 8)))
        atomicAdd((unsigned long long*)&s.tie_h[(u >> shift) & 255], (unsigned long long)s.tie_w[i]);
    }
    __syncthreads();
    if (warp_id() == 0) {
      const int l = lane_id();
      long long v[8], sum = 0;
#pragma unroll
      for (int t = 0; t < 8; t++) {
        v[t] = s.tie_h[8 * l + t];
        sum += v[t];
      }
      long long incl = sum;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        long long y = __shfl_up_sync(0xffffffffu, incl, o);
        if (l >= o) incl += y;
      }
      long long run = s.tie_base + incl - sum;
      int cd = -1;
      long long cb = 0;
#pragma unroll
      for (int t = 0; t < 8; t++) {
        if (cd < 0 && v[t] > 0) {
          if (run + v[t] >= T) {
            cd = 8 * l + t;
            cb = run;
          }
          run += v[t];
        }
      }
      unsigned m = __ballot_sync(0xffffffffu, cd >= 0);
      if (m) {
        int src = __ffs(m) - 1;
        int dd = __shfl_sync(0xffffffffu, cd, src);
        long long bb = __shfl_sync(0xffffffffu, cb, src);
        __syncwarp();  // every lane's read of tie_base precedes lane 0's update (racecheck: WAR)
        if (l == 0) {
          s.tie_prefix |= (unsigned long long)dd << shift;
          s.tie_base = bb;
        }
      }
    }
    __syncthreads();
  }
  return (unsigned)s.tie_prefix;
}

// ---------------------------------------------------------------------------
// CTA-cooperative processing of hubs (degree > kBlockDeg): the "block" bucket
// of the degree-bucketed work assignment (thread <= 16 < warp <= 1024 < CTA)
// ---------------------------------------------------------------------------
// sum of (a, b) over the CTA, result in every thread
__device__ __forceinline__ void block_sum2(RefSmem& s, long long& a, long long& b) {
  a = warp_sum(a);
  b = warp_sum(b);
  __syncthreads();
  if (lane_id() == 0) {
    s.red[warp_id()] = a;
    s.red[kWarps + warp_id()] = b;
  }
  __syncthreads();
  a = 0;
  b = 0;
  for (int w = 0; w < (int)(blockDim.x >> 5); w++) {
    a += s.red[w];
    b += s.red[kWarps + w];
  }
  __syncthreads();
}
// CTA-strided walk over u's prefix, 4 entries per thread per round trip
template <class F>
__device__ __forceinline__ void nbrs_block(const Dev& d, int u, F f) {
  long long o;
  int dg;
  vr_ld(d, u, o, dg);
  for (int b = 0; b < dg; b += 4 * (int)blockDim.x) {
    int x[4], w[4];
    uint8_t q[4];
#pragma unroll
    for (int t = 0; t < 4; t++) {
      int i = b + t * (int)blockDim.x + (int)threadIdx.x;
      x[t] = i < dg ? ldro(d.adj + o + i) : -1;
      w[t] = (i < dg && d.adjw) ? ldro(d.adjw + o + i) : 1;
    }
#pragma unroll
    for (int t = 0; t < 4; t++) q[t] = x[t] >= 0 ? ld_part(d.part, x[t]) : (uint8_t)0;
    f(x, w, q);
  }
}
// CTA-strided walk with an early exit: after each chunk the CTA stops as soon
// as any thread's f returned true (used by the round gain: one smaller-ID
// pseudo neighbour blocks the hub, the rest of its 10^3-10^4 entries need
// not be read)
template <class F>
__device__ __forceinline__ void nbrs_block_until(const Dev& d, int u, F f) {
  long long o;
  int dg;
  vr_ld(d, u, o, dg);
  for (int b = 0; b < dg; b += 8 * (int)blockDim.x) {
    int x[8], w[8];
    uint8_t q[8];
#pragma unroll
    for (int t = 0; t < 8; t++) {
      int i = b + t * (int)blockDim.x + (int)threadIdx.x;
      x[t] = i < dg ? ldro(d.adj + o + i) : -1;
      w[t] = (i < dg && d.adjw) ? ldro(d.adjw + o + i) : 1;
    }
#pragma unroll
    for (int t = 0; t < 8; t++) q[t] = x[t] >= 0 ? ld_part(d.part, x[t]) : (uint8_t)0;
    if (__syncthreads_or(f(x, w, q))) return;
  }
}
// hub filter (Alg. 3 L8-24) by a whole CTA; candidates go to `hout`
__device__ void hub_filter(const Dev& d, RefSmem& s, const int32_t* hubs, int nh, uint32_t ep, int* nout,
                           int32_t* hout, long long& scanned, long long& counted) {
  for (int h = blockIdx.x; h < nh; h += gridDim.x) {
    const int u = __ldcg(hubs + h);
    const uint8_t pu = ld_part(d.part, u);  // deleted vertices carry kDel (== !active)
    if (pu == kDel || pu == kPsi || !own(d, u)) continue;  // uniform over the CTA (sharded: owners filter)
    long long in = 0, ex = 0;
    nbrs_block(d, u, [&](const int* x, const int* w, const uint8_t* q) {
#pragma unroll
      for (int t = 0; t < 4; t++)
        if (x[t] >= 0) {
          if (q[t] == pu) in += w[t]; else ex += w[t];
        }
    });
    block_sum2(s, in, ex);
    if (threadIdx.x == 0) {
      path_hit(d.ctl, PA_HUB_FILTER);
      counted++;
      scanned += ldro(&d.vr[u].deg);
      if (ex > in) {
        d.markT[u] = ep;
        d.oldp[u] = pu;
        hout[atomicAdd(nout, 1)] = u;
      }
    }
  }
}

// filter (Alg. 3 L8-24): candidates = listed placed vertices with ext > int;
// pseudo neighbours count as external (Q13); strict > (Q2)
// (vertices stamped markH == hub_ep are left to the CTA-cooperative hub pass)
// nx > 0 (F0): items n .. n + nx of the same pass are xlist[0, nx) (the
// vertices pending since the apply); each one still pending adds 1 to *xcnt
// and is not filtered -- one pass instead of a separate counting loop
template <class Get>
__device__ void filter_pass(const Dev& d, long long n, Get get, int* ncand, int32_t* cand, uint32_t ep,
                            long long& scanned, long long& counted, uint32_t hub_ep = 0, int nx = 0,
                            const int32_t* xlist = nullptr, long long* xcnt = nullptr) {
  // the label doubles as the active flag; hubs of A go to the CTA pass;
  // sharded: the owner filters
  auto pre = [&](int u, long long i) -> int {
    const uint8_t pu = ld_part(d.part, u);
    if (i >= n) {
      *xcnt += pu == kPsi;
      return -1;
    }
    const bool hub = hub_ep && __ldcg(d.markH + u) == hub_ep;
    return (pu == kDel || hub || pu == kPsi || !own(d, u)) ? -1 : (int)pu;
  };
  auto tf = [&](int u, long long, long long o, int dg, int pvv) {
    const uint8_t pu = (uint8_t)pvv;
    counted++;
    long long in = 0, ex = 0;
    nbrs_thread(d, o, dg, [&](int, int w, uint8_t q) {
      if (q == pu) in += w; else ex += w;
      return true;
    });
    scanned += dg;
    bool c = ex > in;
    if (c) {  // stamp + snapshot label: the commit reads it while labels change
      d.markT[u] = ep;
      d.oldp[u] = pu;
    }
    int slot = agg_append(ncand, c);
    if (c) cand[slot] = u;
  };
  auto wf = [&](int u, long long, long long o, int dg, int pvv) {
    const uint8_t pu = (uint8_t)pvv;
    long long in = 0, ex = 0;
    nbrs_warp(d, o, dg, [&](int, int w, uint8_t q) {
      if (q == pu) in += w; else ex += w;
    });
    in = warp_sum(in);
    ex = warp_sum(ex);
    if (lane_id() == 0) {
      counted++;
      scanned += dg;
      if (ex > in) {
        d.markT[u] = ep;
        d.oldp[u] = pu;
        cand[atomicAdd(ncand, 1)] = u;
      }
    }
  };
  foreach_vertex(
      d, n + nx, [&](long long i) { return i < n ? get(i) : __ldcg(xlist + (i - n)); }, pre, tf, wf);
}

// deferred commit to the pseudo-partition (Alg. 3 L25-26) of the candidates
// stamped `ep`: W_p, label, frontier list, and the exact cut delta.  A
// neighbour's snapshot label is its saved label if it is a candidate (its
// current label may already be psi), else its current label.  With `expand`,
// the placed-on-sigma2 neighbours are marked for R2.
//
// np0 > 0 (F1): the same pass also marks the placed neighbours of the np0
// vertices pending since the apply (plist0[0, np0): items nc .. nc + np0 of
// the pass), so the commit chains and the marking chains run side by side on
// different warps instead of one after the other (C2: the marking pass
// alone held the slowest CTA ~10 us past the commit).
__device__ void commit(const Dev& d, RefSmem& s, const RefineArgs& a, int nc, const int32_t* cand, uint32_t ep,
                       bool expand, long long& scanned, long long& cut_acc, int np0 = 0,
                       const int32_t* plist0 = nullptr) {
  Ctl* ctl = d.ctl;
  auto finish = [&](int u, uint8_t pu) {
    acc_add(s.acc, pu, -(long long)vert_w(d.vw, u));
    d.part[u] = kPsi;
    int slot = agg_append(&ctl->npsi[0], true);
    d.psi[0][slot] = u;
  };
  auto pre = [&](int u, long long i) -> int {
    if (i >= nc) return ld_part(d.part, u) == kPsi ? (int)kPsi : -1;  // pending since the apply: mark only
    return __ldcg(d.oldp + u);
  };
  int dmax = 0;  // diagnostics (IGK_DEBUG_ARRIVALS): the heaviest prefix this warp handled
  auto tf = [&](int u, long long i, long long o, int dg, int pvv) {
    scanned += dg;
    dmax = max(dmax, dg | (i >= nc ? 1 << 21 : 0));
    if (i >= nc) {
      mark_nbrs_thread(d, o, dg, a.epN, ep);
      return;
    }
    const uint8_t pu = (uint8_t)pvv;
    long long del = 0;
    for (int i = 0; i < dg; i += kTCc) {
      int x[kTCc], w[kTCc];
      uint8_t q[kTCc];
      unsigned mk[kTCc];
#pragma unroll
      for (int t = 0; t < kTCc; t++) {
        x[t] = (i + t < dg) ? ldro(d.adj + o + i + t) : -1;
        w[t] = (i + t < dg && d.adjw) ? ldro(d.adjw + o + i + t) : 1;
      }
      uint8_t op[kTCc];
      int dgx[kTCc];
#pragma unroll
      for (int t = 0; t < kTCc; t++) {  // label, stamp, saved label (+ expansion: prefix length) in one round trip
        q[t] = x[t] >= 0 ? ld_part(d.part, x[t]) : (uint8_t)0;
        mk[t] = x[t] >= 0 ? __ldcg(d.markT + x[t]) : 0u;
        op[t] = x[t] >= 0 ? __ldcg(d.oldp + x[t]) : (uint8_t)0;
        dgx[t] = (expand && x[t] >= 0) ? ldro(&d.vr[x[t]].deg) : 0;
      }
#pragma unroll
      for (int t = 0; t < kTCc; t++) {
        if (x[t] < 0) continue;
        const bool xc = mk[t] == ep;
        const uint8_t qx = xc ? op[t] : q[t];
        if (qx != kPsi && qx != pu && !(xc && x[t] < u)) del += w[t];
      }
      if (expand) mark_chunk<kTCc>(d, x, q, a.epN, ep, mk, dgx);
    }
    if (own(d, u)) cut_acc -= del;  // sharded: the owner (full prefix) keeps the cut delta
    finish(u, pu);
  };
  auto wf = [&](int u, long long i, long long o, int dg, int pvv) {
    if (lane_id() == 0) scanned += dg;
    dmax = max(dmax, dg + (i >= nc ? 0 : 1 << 20));  // + 2^20: a commit (not a mark) on the warp path
    if (i >= nc) {
      mark_nbrs_warp(d, o, dg, a.epN, ep);
      return;
    }
    const uint8_t pu = (uint8_t)pvv;
    long long del = 0;
    for (int b = 0; b < dg; b += kWB) {
      int x[kWU], w[kWU];
      uint8_t q[kWU];
      unsigned mk[kWU];
#pragma unroll
      for (int t = 0; t < kWU; t++) {
        int i = b + t * 32 + lane_id();
        x[t] = i < dg ? ldro(d.adj + o + i) : -1;
        w[t] = (i < dg && d.adjw) ? ldro(d.adjw + o + i) : 1;
      }
      uint8_t op[kWU];
      int dgx[kWU];
#pragma unroll
      for (int t = 0; t < kWU; t++) {
        q[t] = x[t] >= 0 ? ld_part(d.part, x[t]) : (uint8_t)0;
        mk[t] = x[t] >= 0 ? __ldcg(d.markT + x[t]) : 0u;
        op[t] = x[t] >= 0 ? __ldcg(d.oldp + x[t]) : (uint8_t)0;
        dgx[t] = (expand && x[t] >= 0) ? ldro(&d.vr[x[t]].deg) : 0;
      }
#pragma unroll
      for (int t = 0; t < kWU; t++) {
        if (x[t] < 0) continue;
        const bool xc = mk[t] == ep;
        const uint8_t qx = xc ? op[t] : q[t];
        if (qx != kPsi && qx != pu && !(xc && x[t] < u)) del += w[t];
      }
      if (expand) mark_chunk<kWU>(d, x, q, a.epN, ep, mk, dgx);
    }
    del = warp_sum(del);
    if (lane_id() == 0) {
      if (own(d, u)) cut_acc -= del;
      finish(u, pu);
    }
  };
  foreach_vertex(
      d, (long long)nc + np0, [&](long long i) { return i < nc ? __ldcg(cand + i) : __ldcg(plist0 + (i - nc)); },
      pre, tf, wf);
  if (d.dbg && expand) {  // per warp: end time, heaviest prefix (igk_debug_arrivals which = 2)
#pragma unroll
    for (int o2 = 16; o2; o2 >>= 1) dmax = max(dmax, __shfl_xor_sync(0xffffffffu, dmax, o2));
    const long long wi = (long long)blockIdx.x * (blockDim.x >> 5) + warp_id();
    if (lane_id() == 0 && wi < 4096) {
      d.dbg[kDbgWarp + wi] = gtimer();
      d.dbg[kDbgWarp + 4096 + wi] = (unsigned long long)dmax;
    }
  }
}

// commit of hub candidates by a whole CTA each (same arithmetic as commit());
// committed hubs are stamped and listed for CTA-cooperative rounds
__device__ void hub_commit(const Dev& d, RefSmem& s, const RefineArgs& a, const int32_t* hubs, int nh, uint32_t ep,
                           bool expand, long long& scanned, long long& cut_acc) {
  Ctl* ctl = d.ctl;
  for (int h = blockIdx.x; h < nh; h += gridDim.x) {
    const int u = __ldcg(hubs + h);
    const uint8_t pu = __ldcg(d.oldp + u);
    long long del = 0, dummy = 0;
    nbrs_block(d, u, [&](const int* x, const int* w, const uint8_t* q) {
      unsigned mk[4];
      uint8_t op[4];
#pragma unroll
      for (int t = 0; t < 4; t++) {
        mk[t] = x[t] >= 0 ? __ldcg(d.markT + x[t]) : 0u;
        op[t] = x[t] >= 0 ? __ldcg(d.oldp + x[t]) : (uint8_t)0;
      }
#pragma unroll
      for (int t = 0; t < 4; t++) {
        if (x[t] < 0) continue;
        const bool xc = mk[t] == ep;
        const uint8_t qx = xc ? op[t] : q[t];
        if (qx != kPsi && qx != pu && !(xc && x[t] < u)) del += w[t];
      }
      if (expand) mark_chunk<4>(d, x, q, a.epN, ep);
    });
    block_sum2(s, del, dummy);
    if (threadIdx.x == 0) {
      path_hit(ctl, PA_HUB_COMMIT);
      scanned += ldro(&d.vr[u].deg);
      if (own(d, u)) cut_acc -= del;
      atomic_add_ll(&ctl->Wp[pu], -(long long)vert_w(d.vw, u));
      d.part[u] = kPsi;
      d.psi[0][atomicAdd(&ctl->npsi[0], 1)] = u;
      d.markH[u] = a.epF;  // rounds: handled by a whole CTA
      d.hubP[atomicAdd(&ctl->nhubP, 1)] = u;
    }
    __syncthreads();
  }
}

// better(a, b) on (conn desc, W_p asc, p asc)  (reading Q6)
__device__ __forceinline__ bool better(long long ca, int pa, long long cb, int pb, const long long* Wr) {
  if (pb < 0) return true;
  if (ca != cb) return ca > cb;
  if (Wr[pa] != Wr[pb]) return Wr[pa] < Wr[pb];
  return pa < pb;
}

// ---------------------------------------------------------------------------
// R4 rounds (Alg. 4) until the pseudo-partition is empty,
// all CTAs with grid barriers.
// ---------------------------------------------------------------------------
struct RoundState {
  int cur = 0;
  long long rounds = 0, rounds_all = 0, applied_tot = 0, deferred_tot = 0;
};
template <bool kSh>
__device__ void run_rounds(const Dev& d, const RefineArgs& a, RefSmem& s, cg::grid_group& grid, long long c,
                           int exact_shift_id, RoundState& rs, long long& scanned, long long& cut_acc,
                           const ShardArgs& sh_in, PhaseWork& pw_) {
  // kSh = false: the single-GPU kernels, all sharding code compiled out.
  // kSh: ONE round per launch, on the canonical pending list d.psi[1] (sorted
  // by ID, the same on every rank, positions fixed for all rounds): kShGain
  // writes the owned moves' records d.recs[j]; kShFinish installs every
  // rank's records (all-reduced) and takes + applies the balanced prefix.
  ShardArgs sh = sh_in;
  if (!kSh) sh.mode = kModeFull;
  const bool sh_gain = kSh && sh.mode == kShGain, sh_fin = kSh && sh.mode == kShFinish;
  Ctl* ctl = d.ctl;
  const int k = d.k;
  const long long tid = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  int& cur = rs.cur;
  long long& rounds = rs.rounds;
  long long& rounds_all = rs.rounds_all;
  long long& applied_tot = rs.applied_tot;
  long long& deferred_tot = rs.deferred_tot;
  const int nhp = ldv(&ctl->nhubP);  // final after F3: hubs pending in the rounds
  auto round_sync = [&](int id) {  // per-round arrival slots 20 + 2r (gain), 21 + 2r (apply)
    const bool per_round = (id == 208 || id == 209) && rounds_all < 40;
    arrive_stamp(d.dbg, per_round ? 20 + 2 * (int)rounds_all + (id - 208) : id % 100);
    grid.sync();
    stamp_phase(ctl, id);
  };
  while (true) {
    const int np = kSh ? (int)sh.np : ldv(&ctl->npsi[cur]);
    if (np == 0) break;
    const int nxt = cur == 1 ? 2 : 1;
    const int32_t* plist = kSh ? d.psi[1] : d.psi[cur];
    int32_t* pnext = d.psi[nxt];
    const int r3 = (int)(rounds_all % 3), r3n = (int)((rounds_all + 1) % 3);
    // round-start snapshot of W_p (Q14) and the lightest part (zero-conn choice)
    for (int p = threadIdx.x; p < k; p += blockDim.x) s.Wr[p] = ldv(&ctl->Wp[p]);
    __syncthreads();
    if (threadIdx.x == 0) {
      int b = 0;
      for (int p = 1; p < k; p++)
        if (s.Wr[p] < s.Wr[b]) b = p;
      s.best0 = b;
    }
    __syncthreads();
    if (tid == 0 && !sh_gain) {
      ctl->npsi[nxt] = 0;
      ctl->applied3[r3n] = 0;
      ctl->selected3[r3n] = 0;
      if (kSh) ctl->rs_pending = 0;  // counted by the apply below (after barrier 208)
    }
    // -- gain: selection + best part, one adjacency pass per vertex
    long long sel_cnt = 0;
    if (!sh_fin) {  // (the finish launch of a sharded round starts at the install)
    if (!kSh) rr_for(k, [&](long long p) { ctl->tot3[r3n][p] = 0; });
    auto emit_move = [&](long long j, int u, int best, long long g, long long pwv, bool imbal) {
      int d0 = 255 - (int)min(g, 255ll);
      if (kSh) {  // the record at the vertex's canonical position; installed by every rank in kShFinish
        const int4 rec = make_int4(u + 1, (int)(0x80000000u | ((unsigned)d0 << 8) | (unsigned)best | (imbal ? 1u << 30 : 0u)),
                                   (int)g, (int)pwv);
        if (d.p2p_n) {  // NEXT-3: straight into every rank's buffer (peer stores over NVLink)
          for (int q = 0; q < d.p2p_n; q++) d.p2p_recs[q][j] = rec;
        } else {
          d.recs[j] = rec;
        }
        return;
      }
      d.tgt[u] = (uint8_t)best;
      d.gain[u] = (int)g;
      d.pw[u] = (int)pwv;
      d.meta[j] = 0x80000000u | ((unsigned)d0 << 8) | (unsigned)best;  // j: list position
      long long w = vert_w(d.vw, u);
      // lanes with the same (part, digit) / part combine first: one global
      // atomic per distinct key per warp (the round's hot histogram cells)
      acc_add(d.hist0, best * kDigits + d0, w);
      acc_add(ctl->tot3[r3], best, w);
      if (imbal) {
        ctl->st[ST_IMBAL] = 1;
        path_hit(ctl, PA_WFALLBACK);
      }
    };
    auto emit_move_v = [&](int u, int best, long long g, long long pwv, bool imbal) {
      int d0 = 255 - (int)min(g, 255ll);
      d.tgt[u] = (uint8_t)best;
      d.gain[u] = (int)g;
      d.pw[u] = (int)pwv;
      d.metav[u] = 0x80000000u | ((unsigned)d0 << 8) | (unsigned)best;
      long long w = vert_w(d.vw, u);
      atomic_add_ll(d.hist0 + (long long)best * kDigits + d0, w);
      atomic_add_ll(&ctl->tot3[r3][best], w);
      if (imbal) {
        ctl->st[ST_IMBAL] = 1;
        path_hit(ctl, PA_WFALLBACK);
      }
    };
    auto get = [&](long long i) {
      int u = __ldcg(plist + i);
      if (u < 0 && !kSh) d.meta[i] = 0;
      return u;
    };
    auto pre = [&](int u, long long i) -> int {  // issued together with the vertex record
      const uint8_t pu = ld_part(d.part, u);
      const bool act = pu != kDel;  // the label doubles as the active flag
      if (kSh) return (act && pu == kPsi && own(d, u)) ? (int)pu : -1;  // hubs: warp path; others: their owners
      const bool hub = __ldcg(d.markH + u) == a.epF;
      if (!act || pu != kPsi) {
        d.meta[i] = 0;
        return -1;
      }
      if (hub) {  // CTA-cooperative below; its record is kept per vertex in metav
        d.meta[i] = kMetaHub;
        return -1;
      }
      return (int)pu;
    };
    // thread bucket (degree <= kThreadDeg, one load round trip): the whole
    // prefix sits in registers (static indices only -- no local-memory
    // tally); conn(u, p) for each neighbour's label p is a register-only
    // sum over the <= 16 slots, so every candidate part is evaluated
    // exactly as the warp / CTA buckets do it (reading Q6).
    auto tf = [&](int u, long long j, long long o, int dg, int) {
      const long long vwu = vert_w(d.vw, u);
      scanned += dg;
      int x[kThreadDeg], w[kThreadDeg];
      uint8_t q[kThreadDeg];
#pragma unroll
      for (int t = 0; t < kThreadDeg; t++) {
        x[t] = t < dg ? ldro(d.adj + o + t) : -1;
        w[t] = (t < dg && d.adjw) ? ldro(d.adjw + o + t) : 1;
      }
#pragma unroll
      for (int t = 0; t < kThreadDeg; t++) q[t] = x[t] >= 0 ? ld_part(d.part, x[t]) : kDel;  // tombstone: no part
      bool sel = true;
      long long pwv = 0;
#pragma unroll
      for (int t = 0; t < kThreadDeg; t++) {
        if (q[t] == kPsi && x[t] < u) sel = false;  // a smaller-ID pseudo neighbour moves first (Alg. 4 L8)
        if (q[t] < kDel) pwv += w[t];
      }
      if (!sel) {
        if (!kSh) d.meta[j] = 0;
        return;
      }
      auto conn_of = [&](int p) {
        int cc = 0;
#pragma unroll
        for (int t = 0; t < kThreadDeg; t++) cc += q[t] == p ? w[t] : 0;
        return (long long)cc;
      };
      int best = -1;
      long long bc = -1;
#pragma unroll
      for (int t = 0; t < kThreadDeg; t++) {
        const int p = q[t];
        if (p >= kDel || s.Wr[p] + vwu > c) continue;  // tombstone / pseudo / ineligible (Q3)
        const long long cc = conn_of(p);
        if (better(cc, p, bc, best, s.Wr)) {
          best = p;
          bc = cc;
        }
      }
      bool imbal = false;
      if (best < 0) {  // lightest part: eligible => zero connectivity; else fallback (Q8)
        best = s.best0;
        bc = 0;
        if (s.Wr[best] + vwu > c) {
          imbal = true;
          bc = conn_of(best);
        }
      }
      sel_cnt++;
      emit_move(j, u, best, bc, pwv, imbal);
    };
    auto wf = [&](int u, long long j, long long o, int dg, int) {
      const long long vwu = vert_w(d.vw, u);
      int* wc = s.wconn[warp_id()];
      if (lane_id() == 0) {
        scanned += dg;
        path_hit(ctl, PA_WARP_GAIN);
      }
      bool lb = false;
      long long pwv = 0;
      nbrs_warp_until(
          d, o, dg,
          [&](int x, int w, uint8_t q) {
            if (q == kPsi) {
              lb |= x < u;
            } else {
              atomicAdd(wc + q, w);
              pwv += w;
            }
          },
          [&]() { return lb; });  // blocked (Alg. 4 L8-10): the rest of the prefix is not needed
      const bool blocked = __any_sync(0xffffffffu, lb);
      pwv = warp_sum(pwv);
      __syncwarp();
      long long bc = -1;
      int best = -1;
      if (!blocked) {
        for (int p = lane_id(); p < k; p += 32) {
          if (s.Wr[p] + vwu > c) continue;
          long long cc = wc[p];
          if (better(cc, p, bc, best, s.Wr)) {
            best = p;
            bc = cc;
          }
        }
#pragma unroll
        for (int off = 16; off > 0; off >>= 1) {
          long long oc = __shfl_xor_sync(0xffffffffu, bc, off);
          int op = __shfl_xor_sync(0xffffffffu, best, off);
          if (op >= 0 && better(oc, op, bc, best, s.Wr)) {
            bc = oc;
            best = op;
          }
        }
      }
      bool imbal = false;
      if (!blocked && best < 0) {
        best = s.best0;
        bc = wc[best];
        imbal = true;
      }
      __syncwarp();
      for (int p = lane_id(); p < k; p += 32) wc[p] = 0;
      __syncwarp();
      if (lane_id() == 0) {
        if (blocked) {
          if (!kSh) d.meta[j] = 0;
        } else {
          sel_cnt++;
          emit_move(j, u, best, bc, pwv, imbal);
        }
      }
    };
    foreach_vertex(d, np, get, pre, tf, wf);
    if (!kSh) {  // hubs in the pseudo-partition: one CTA each
      int* conn = s.wconn[0];
      for (int h = blockIdx.x; h < nhp; h += gridDim.x) {
        const int u = __ldcg(d.hubP + h);
        if (ld_part(d.part, u) != kPsi) continue;  // uniform: placed earlier (or deleted)
        const long long vwu = vert_w(d.vw, u);
        __syncthreads();
        for (int p = threadIdx.x; p < 256; p += blockDim.x) conn[p] = 0;
        __syncthreads();
        bool lb = false;
        long long pwv = 0, dummy = 0;
        nbrs_block_until(d, u, [&](const int* x, const int* w, const uint8_t* q) {
#pragma unroll
          for (int t = 0; t < 8; t++) {
            if (x[t] < 0) continue;
            if (q[t] == kPsi) {
              lb |= x[t] < u;
            } else {
              atomicAdd(conn + q[t], w[t]);
              pwv += w[t];
            }
          }
          return lb;  // blocked (Alg. 4 L8-10): the rest of the prefix is not needed
        });
        const bool blocked = __syncthreads_or(lb);
        block_sum2(s, pwv, dummy);
        long long bc = -1;
        int best = -1;
        if (!blocked) {
          for (int p = threadIdx.x; p < k; p += blockDim.x) {
            if (s.Wr[p] + vwu > c) continue;
            if (better(conn[p], p, bc, best, s.Wr)) {
              best = p;
              bc = conn[p];
            }
          }
#pragma unroll
          for (int off = 16; off > 0; off >>= 1) {
            long long oc = __shfl_xor_sync(0xffffffffu, bc, off);
            int op = __shfl_xor_sync(0xffffffffu, best, off);
            if (op >= 0 && better(oc, op, bc, best, s.Wr)) {
              bc = oc;
              best = op;
            }
          }
          if (lane_id() == 0) {
            s.red[warp_id()] = bc;
            s.red[kWarps + warp_id()] = best;
          }
        }
        __syncthreads();
        if (threadIdx.x == 0) {
          path_hit(ctl, PA_HUB_GAIN);
          if (blocked) {
            d.metav[u] = 0;
          } else {
            bc = -1;
            best = -1;
            for (int w = 0; w < (int)(blockDim.x >> 5); w++) {
              int op = (int)s.red[kWarps + w];
              if (op >= 0 && better(s.red[w], op, bc, best, s.Wr)) {
                bc = s.red[w];
                best = op;
              }
            }
            bool imbal = false;
            if (best < 0) {  // E(u) empty (Q8)
              best = s.best0;
              bc = conn[best];
              imbal = true;
            }
            sel_cnt++;
            scanned += ldro(&d.vr[u].deg);
            emit_move_v(u, best, bc, pwv, imbal);
          }
        }
        __syncthreads();
        // conn is warp 0's histogram: the warp path expects it zeroed
        for (int p = threadIdx.x; p < 256; p += blockDim.x) conn[p] = 0;
        __syncthreads();
      }
    }
    if (!kSh) {
      long long sc = warp_sum(sel_cnt);
      if (lane_id() == 0 && sc) atomicAdd(&ctl->selected3[r3], (int)sc);
    }
    }  // gain
    if (sh_gain) return;  // the host all-reduces the move records
    if (sh_fin) {
      // install every rank's move of this round (records all-reduced: at most
      // one rank wrote each position) exactly as the single-GPU gain does;
      // tot3[r3] was zeroed by the previous finish (or the last epilogue)
      rr_for(np, [&](long long j) {
        const int4 e = __ldcg(d.recs + j);
        if (e.x == 0) {
          d.meta[j] = 0;
          return;
        }
        const int u = e.x - 1;
        const unsigned m = (unsigned)e.y & ~(1u << 30);
        const int best = (int)(m & 255u), d0 = (int)((m >> 8) & 255u);
        d.tgt[u] = (uint8_t)best;
        d.gain[u] = e.z;
        d.pw[u] = e.w;
        d.meta[j] = m;
        const long long w = vert_w(d.vw, u);
        acc_add(d.hist0, best * kDigits + d0, w);
        acc_add(ctl->tot3[r3], best, w);
        atomicAdd(&ctl->selected3[r3], 1);
        if ((unsigned)e.y & (1u << 30)) {
          ctl->st[ST_IMBAL] = 1;
          path_hit(ctl, PA_WFALLBACK);
        }
      });
    }
    PHASE_FLUSH(PH_GAIN, np);
    round_sync(208);

    // -- balanced prefix: T_p = c - W_p + 1; K* = min over parts of the first
    //    move whose running weight in (#nbr desc, ID asc) order exceeds c.
    for (int p = threadIdx.x; p < k; p += blockDim.x) {
      long long T = c - s.Wr[p] + 1;
      s.sel.T[p] = T;
      s.sel.used[p] = ldv(&ctl->tot3[r3][p]) >= T;
    }
    __syncthreads();
    auto items = [&](long long j, int& p, int& d0, unsigned long long& R, long long& w) {
      unsigned m = __ldcg(d.meta + j);
      const int u = __ldcg(plist + j);
      if (m == kMetaHub) m = __ldcg(d.metav + u);
      if (!(m & 0x80000000u)) return false;
      p = (int)(m & 255u);
      d0 = (int)((m >> 8) & 255u);
      R = d0 ? (unsigned long long)u
             : (((unsigned long long)(0x7fffffffu - (unsigned)__ldcg(d.gain + u))) << 32) | (unsigned)u;
      w = vert_w(d.vw, u);
      return true;
    };
    sel_digit0(d, s.sel, [](int d0) { return d0 != 0; }, exact_shift_id);
    if (s.sel.nactive > 0) {
      // tie groups (moves of an overflowing part with its threshold digit 0)
      rr_for(np, [&](long long j) {
        int p, d0;
        unsigned long long R;
        long long w;
        bool in = items(j, p, d0, R, w) && s.sel.active[p] && d0 == s.sel.d0[p];
        int slot = agg_append(&ctl->ntie, in);
        if (in) {
          d.r3list[slot] = make_int2(__ldcg(plist + j), p | ((int)w << 8));
          atomicAdd(&ctl->tiecnt[p], 1);
        }
      });
      round_sync(212);
      const int ntie = ldv(&ctl->ntie);
      bool local_ok = true;
      int nexact = 0, n64 = 0;
      for (int p = 0; p < k; p++)
        if (s.sel.active[p]) {
          local_ok &= s.sel.exact[p] && ldv(&ctl->tiecnt[p]) <= kTieMax;
          nexact += s.sel.exact[p] != 0;
          n64 += s.sel.exact[p] == 0;
        }
      if (tid == 0) {
        if (nexact) path_hit(ctl, PA_KEY_EXACT, nexact);
        if (n64) path_hit(ctl, PA_KEY64, n64);
        if (!local_ok) path_hit(ctl, PA_TIE_GRID);
      }
      if (local_ok) {
        // one CTA per overflowing part finishes its select in shared memory
        for (int p = blockIdx.x; p < k; p += gridDim.x) {
          if (!s.sel.active[p]) continue;
          if (threadIdx.x == 0) s.tie_n = 0;
          __syncthreads();
          for (int i = threadIdx.x; i < ntie; i += blockDim.x) {
            int2 e = __ldcg(d.r3list + i);
            if ((e.y & 255) == p) {
              int q = atomicAdd(&s.tie_n, 1);
              s.tie_u[q] = e.x;
              s.tie_w[q] = e.y >> 8;
            }
          }
          __syncthreads();
          unsigned key = block_select_ids(s, s.tie_n, s.sel.base[p], s.sel.T[p]);
          if (threadIdx.x == 0) {
            ctl->kres[p] = key;
            path_hit(ctl, PA_TIE_CTA);
          }
          __syncthreads();
        }
        round_sync(213);
        for (int p = threadIdx.x; p < k; p += blockDim.x)
          if (s.sel.active[p]) {
            s.sel.prefix[p] = ldv((const long long*)&ctl->kres[p]);
            s.sel.active[p] = 0;
          }
        __syncthreads();
      } else {  // fallback: grid-wide radix passes over the tie buffer only
        auto tie_items = [&](long long j, int& p, int& d0, unsigned long long& R, long long& w) {
          int2 e = __ldcg(d.r3list + j);
          p = e.y & 255;
          w = e.y >> 8;
          d0 = s.sel.d0[p];
          R = s.sel.exact[p] ? (unsigned long long)e.x
                             : (((unsigned long long)(0x7fffffffu - (unsigned)__ldcg(d.gain + e.x))) << 32) |
                                   (unsigned)e.x;
          return true;
        };
        sel_passes(d, s.sel, grid, ntie, tie_items);
      }
    }
    int kd = 1 << 30;
    unsigned long long kr = ~0ull;
    for (int p = 0; p < k; p++) {
      if (s.sel.used[p] && s.sel.found[p] && key_less(s.sel.d0[p], s.sel.prefix[p], kd, kr)) {
        kd = s.sel.d0[p];
        kr = s.sel.prefix[p];
      }
    }
    // -- apply the prefix (moves with key < K*); the rest stay pseudo
    long long app = 0;
    rr_for(np, [&](long long j) {
      // the list entry and its move record in one round trip, then the
      // vertex's words (placed-neighbour weight, gain) in the next
      const int u = __ldcg(plist + j);
      unsigned m = __ldcg(d.meta + j);
      if (u < 0) return;
      if (m == kMetaHub) m = __ldcg(d.metav + u);
      const bool sel = (m & 0x80000000u) != 0;
      const int pwu = sel ? __ldcg(d.pw + u) : 0;
      const int gu = sel ? __ldcg(d.gain + u) : 0;
      bool keep = true;
      if (sel) {
        const int p = (int)(m & 255u), d0 = (int)((m >> 8) & 255u);
        const unsigned long long R =
            d0 ? (unsigned long long)u : (((unsigned long long)(0x7fffffffu - (unsigned)gu)) << 32) | (unsigned)u;
        if (key_less(d0, R, kd, kr)) {
          keep = false;
          d.part[u] = (uint8_t)p;
          acc_add(s.acc, p, vert_w(d.vw, u));
          if (!kSh || own(d, u))  // sharded: the owner keeps this delta in its partial cut
            cut_acc += (long long)pwu - gu;  // independent set: exact
          app++;
        }
      } else if (ld_part(d.part, u) != kPsi) {
        keep = false;  // stale entry (deleted before this refine / placed in an earlier round)
      }
      if (kSh) {  // canonical list: positions stay; count what is left pending
        agg_append(&ctl->rs_pending, keep);
        return;
      }
      int slot = agg_append(&ctl->npsi[nxt], keep);
      if (keep) pnext[slot] = u;
    });
    flush_acc(s, ctl->Wp, k);
    {
      long long sa = warp_sum(app);
      if (lane_id() == 0 && sa) atomicAdd(&ctl->applied3[r3], (int)sa);
    }
    rr_for((long long)k * kDigits, [&](long long t) { d.hist0[t] = 0; });
    rr_for(k, [&](long long p) { ctl->tiecnt[p] = 0; });
    if (kSh) rr_for(k, [&](long long p) { ctl->tot3[r3n][p] = 0; });  // the next finish accumulates there
    if (tid == 0) ctl->ntie = 0;
    sel_clear(d, s.sel);
    PHASE_FLUSH(PH_MOVE, np);
    round_sync(209);
    const int napp = ldv(&ctl->applied3[r3]), nsel = ldv(&ctl->selected3[r3]);
    if (napp == 0 && nsel > 0) {
      // L = 0: force the first move (reading Q8); it is the threshold item K*
      const int uf = (int)(kr & 0xffffffffu);
      if (!kSh) {
        const int nn = ldv(&ctl->npsi[nxt]);
        rr_for(nn, [&](long long j) {
          if (__ldcg(pnext + j) == uf) pnext[j] = -1;
        });
      }
      if (tid == 0) {
        int p = __ldcg(d.tgt + uf);
        d.part[uf] = (uint8_t)p;
        atomic_add_ll(&ctl->Wp[p], vert_w(d.vw, uf));
        if (kSh) ctl->rs_pending -= 1;
        if (!kSh || own(d, uf)) atomic_add_ll(&ctl->cut, (long long)__ldcg(d.pw + uf) - __ldcg(d.gain + uf));
        ctl->st[ST_IMBAL] = 1;
        path_hit(ctl, PA_FORCED_L0);
      }
      round_sync(210);
    }
    const int napp2 = (napp == 0 && nsel > 0) ? 1 : napp;
    if (nsel > 0) {
      rounds++;
      applied_tot += napp2;
      deferred_tot += nsel - napp2;
    }
    for (int p = threadIdx.x; p < 256; p += blockDim.x) s.sel.used[p] = 0;
    __syncthreads();
    cur = nxt;
    rounds_all++;
    if (sh_fin) return;  // one round per sharded finish launch
  }

}

// NEXT-1 global boundary refinement: every active placed vertex with
// adj_ext != 0 (a pseudo neighbour is external, reading Q13) joins A on the
// labels as they stand (reading B1).  A full-store scan: 32 consecutive
// vertices per warp (per-vertex arrays read coalesced), each thread walks its
// own prefix with int4 loads and stops at the first external neighbour;
// prefixes longer than kBndHeavy are walked by the whole warp.
constexpr int kBndHeavy = 32;
__device__ __forceinline__ void boundary_mark(const Dev& d, uint32_t epA) {
  const long long n = ldv(&d.ctl->n_total);
  const int lane = lane_id();
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (long long base = (long long)blockIdx.x * blockDim.x + (threadIdx.x & ~31); base < n; base += stride) {
    const long long v = base + lane;
    bool placed = false;
    uint8_t pv = kPsi;
    int dg = 0;
    long long o = 0;
    if (v < n) {
      pv = ld_part(d.part, v);
      placed = pv != kDel && pv != kPsi;
      if (placed) {
        vr_ld(d, v, o, dg);
      }
    }
    bool bnd = false;
    const bool heavy = placed && dg > kBndHeavy;
    if (placed && !heavy) {
      const int4* a4 = reinterpret_cast<const int4*>(d.adj + o);
      for (int i = 0; i < dg && !bnd; i += 8) {  // two int4 per round trip, then 8 label gathers
        int4 a0 = ldro(a4 + (i >> 2));
        int4 a1 = (i + 4 < dg) ? ldro(a4 + (i >> 2) + 1) : make_int4(-1, -1, -1, -1);
        const int xs[8] = {a0.x, a0.y, a0.z, a0.w, a1.x, a1.y, a1.z, a1.w};
        uint8_t qs[8];
#pragma unroll
        for (int t = 0; t < 8; t++) qs[t] = (i + t < dg && xs[t] >= 0) ? ld_part(d.part, xs[t]) : pv;
#pragma unroll
        for (int t = 0; t < 8; t++) bnd |= qs[t] != pv;
      }
    }
    unsigned hm = __ballot_sync(0xffffffffu, heavy);
    while (hm) {
      const int src = __ffs(hm) - 1;
      hm &= hm - 1;
      const long long ho = __shfl_sync(0xffffffffu, o, src);
      const int hd = __shfl_sync(0xffffffffu, dg, src);
      const uint8_t hp = (uint8_t)__shfl_sync(0xffffffffu, (int)pv, src);
      bool hb = false;
      for (int b = 0; b < hd && !hb; b += 256) {
        int x[8];
#pragma unroll
        for (int t = 0; t < 8; t++) {
          int i = b + 32 * t + lane;
          x[t] = i < hd ? ldro(d.adj + ho + i) : -1;
        }
        bool e = false;
#pragma unroll
        for (int t = 0; t < 8; t++) e |= x[t] >= 0 && ld_part(d.part, x[t]) != hp;
        hb = __any_sync(0xffffffffu, e);
      }
      if (lane == src) bnd = hb;
    }
    if (bnd) mark_affected(d, (int)v, epA, dg);
  }
}

// Sharded refine helpers.  Every set bit u of the all-reduced candidate
// bitmap joins the replicated candidate list: stamped `ep`, its label saved,
// hubs (by their LOCAL prefix length: the commit walks the local prefix)
// listed apart.  sh_publish sets the bits of this rank's candidates.
__device__ void sh_extract(const Dev& d, long long nwords, uint32_t ep, int* ncand, int32_t* cand, int* nhub,
                           int32_t* hubs) {
  rr_for(nwords, [&](long long w) {
    unsigned long long b = __ldcg(d.bm + w);
    while (b) {
      const int bit = __ffsll((long long)b) - 1;
      b &= b - 1;
      const int u = (int)(w * 64 + bit);
      d.markT[u] = ep;
      d.oldp[u] = ld_part(d.part, u);
      if (ldro(&d.vr[u].deg) > kBlockDeg) hubs[atomicAdd(nhub, 1)] = u;
      else cand[atomicAdd(ncand, 1)] = u;
    }
  });
}
__device__ void sh_publish(const Dev& d, int n, const int32_t* cand, int nh, const int32_t* hubs) {
  rr_for(n + nh, [&](long long i) {
    const int u = i < n ? __ldcg(cand + i) : __ldcg(hubs + (i - n));
    atomicOr((unsigned long long*)d.bm + (u >> 6), 1ull << (u & 63));
  });
}
__device__ void sh_clear_bm(const Dev& d, long long nwords) {
  rr_for(nwords, [&](long long w) { d.bm[w] = 0; });
}

// Returns true (on every CTA) iff the epilogue ran; the unsharded epilogue
// then also posted the completion notice (publish_copy), so the kernel must
// not call publish() again.
template <bool kSh>
__device__ __forceinline__ bool refine_body(const Dev& d, const RefineArgs& a, cg::grid_group& grid, RefSmem& s,
                                            const ShardArgs& sh) {
  Ctl* ctl = d.ctl;
  const int k = d.k;
  const long long tid = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  const int mode = kSh ? sh.mode : (int)kModeFull;
  if (!kSh && a.after_apply && (ldv(&ctl->err_idx) != kNoErr || ldv(&ctl->err_nomem) != 0)) {
    if (tid == 0) ctl->refine_skipped = 1;  // uniform exit: nothing was modified
    return false;
  }
  if (tid == 0 && (mode == kModeFull || mode == kShF0)) {
    ctl->refine_skipped = 0;
    ctl->n_delta = 0;  // appended only after the last round (many barriers later)
    if (kSh) ctl->rs_rounds = ctl->rs_rounds_all = ctl->rs_applied = ctl->rs_deferred = 0;
  }
  const long long c = cap_of(ldv(&ctl->W), a.e_ppm, k);
  const int exact_shift_id = ((d.idbits + 7) / 8) * 8 - 8;

  for (int p = threadIdx.x; p < 256; p += blockDim.x) {
    s.acc[p] = 0;
    s.sel.used[p] = 0;
    s.sel.active[p] = 0;
  }
  for (int t = threadIdx.x; t < kWarps * 256; t += blockDim.x) (&s.wconn[0][0])[t] = 0;
  __syncthreads();

  if (tid == 0) ctl->nph = 0;
  stamp_phase(ctl, 200);
  arrive_stamp(d.dbg, 0);
  long long scanned = 0, counted = 0, cnt_ins = 0, cut_acc = 0;
  PhaseWork pw_;
  auto flush_partial = [&]() {  // sharded launches: per-kernel accumulators to the control block
    block_atomic_add(&ctl->cut, cut_acc, s.red);
    block_atomic_add(&ctl->st[ST_SCANNED], scanned, s.red);
  };
  const long long nwords = kSh ? (ldv(&ctl->n_total) + 63) / 64 : 0;
  // ---- R3: balance restoration (reading Q9) ----------------------------------------
  // the (int - ext, id) keys of every vertex of an overweight part on sigma3,
  // then the weighted select of each part's eviction threshold + commit
  auto r3_setup = [&]() {
    bool any = false;
    for (int p = 0; p < k; p++) any |= ldv(&ctl->Wp[p]) > c;
    if (any) {
      for (int p = threadIdx.x; p < k; p += blockDim.x) {
        long long wp = ldv(&ctl->Wp[p]);
        s.sel.used[p] = wp > c;
        s.sel.T[p] = wp - c;
      }
    }
    __syncthreads();
    return any;
  };
  auto r3_emit = [&](int v, uint8_t p, long long loss) {
    int d0 = (int)max(0ll, min(255ll, loss + 128));
    atomic_add_ll(d.hist0 + (long long)p * kDigits + d0, vert_w(d.vw, v));
    int slot = atomicAdd(&ctl->nr3, 1);
    d.r3list[slot] = make_int2(v, (int)loss);
  };
  auto r3_select_evict_commit = [&]() {
      const int nr3 = ldv(&ctl->nr3);
      auto items = [&](long long j, int& p, int& d0, unsigned long long& R, long long& w) {
        int2 e = __ldcg(d.r3list + j);
        p = ld_part(d.part, e.x);
        d0 = max(0, min(255, e.y + 128));
        bool ex = d0 != 0 && d0 != 255;
        R = ex ? (unsigned long long)e.x
               : (((unsigned long long)((long long)e.y + 0x80000000ll)) << 32) | (unsigned)e.x;
        w = vert_w(d.vw, e.x);
        return true;
      };
      weighted_select(d, s.sel, grid, [](int d0) { return d0 != 0 && d0 != 255; }, exact_shift_id, nr3, items);
      if (tid == 0) {
        int n64 = 0;
        for (int p = 0; p < k; p++) n64 += s.sel.used[p] && s.sel.found[p] && (s.sel.d0[p] == 0 || s.sel.d0[p] == 255);
        if (n64) path_hit(ctl, PA_R3_KEY64, n64);
      }
      // evict every item with key <= the threshold of its part
      rr_for(nr3, [&](long long j) {
        int p, d0;
        unsigned long long R;
        long long w;
        items(j, p, d0, R, w);
        bool ev = s.sel.found[p] && !key_less(s.sel.d0[p], s.sel.prefix[p], d0, R);
        int slot = agg_append(&ctl->ncand, ev);
        if (ev) {
          int v = __ldcg(d.r3list + j).x;
          d.cand[slot] = v;
          d.markT[v] = a.epE;
          d.oldp[v] = (uint8_t)p;
        }
      });
      sel_clear(d, s.sel);
      GRID_SYNC_STAMPED(ctl, 206);
      const int nc = ldv(&ctl->ncand);
      commit(d, s, a, nc, d.cand, a.epE, false, scanned, cut_acc);
      flush_acc(s, ctl->Wp, k);
      PHASE_FLUSH(PH_R3, nc + nr3);
      if (tid == 0) ctl->st[ST_EVICTED] = nc;
      for (int p = threadIdx.x; p < 256; p += blockDim.x) s.sel.used[p] = 0;
      GRID_SYNC_STAMPED(ctl, 207);
  };
  if (kSh && (mode == kShGain || mode == kShFinish)) {  // one sharded round
    RoundState rs;
    rs.cur = 1;
    rs.rounds = ldv(&ctl->rs_rounds);
    rs.rounds_all = ldv(&ctl->rs_rounds_all);
    rs.applied_tot = ldv(&ctl->rs_applied);
    rs.deferred_tot = ldv(&ctl->rs_deferred);
    run_rounds<kSh>(d, a, s, grid, c, exact_shift_id, rs, scanned, cut_acc, sh, pw_);
    flush_partial();
    grid.sync();  // every CTA read the round state before it is written back
    if (tid == 0 && mode == kShFinish) {
      ctl->rs_rounds = rs.rounds;
      ctl->rs_rounds_all = rs.rounds_all;
      ctl->rs_applied = rs.applied_tot;
      ctl->rs_deferred = rs.deferred_tot;
    }
    return false;
  }
  if constexpr (!kSh) {
    if (a.global) {  // NEXT-1: A |= partition boundary, then the ordinary refine
      boundary_mark(d, a.epA);
      PHASE_FLUSH(PH_BOUNDARY, ldv(&ctl->n_total));
      GRID_SYNC_STAMPED(ctl, 220);
    }
    const int np0 = ldv(&ctl->npsi[0]);  // pending since apply (C1 joins psi[0] beyond np0)
    // F0 + F1 and F2 + F3 are the same two passes (a filter, then the deferred
    // commit of its candidates) over different lists and snapshots, so they
    // run from ONE copy of the code: the second pair executes instructions
    // the first already brought into the instruction caches (the step after
    // a flushed L2 stalls on instruction fetch)
    for (int pass = 0; pass < 2; pass++) {
      const bool p0 = pass == 0;
      {  // ---- F0: R1 filter over A on sigma1 (+ the pending-since-apply count)
         //      F2: R2 filter over N on sigma2
        const int n = ldv(p0 ? &ctl->nA : &ctl->nN);
        const int nh = ldv(p0 ? &ctl->nhubA : &ctl->nhubN);
        const int32_t* list = p0 ? d.Alist : d.Nlist;
        const uint32_t ep = p0 ? a.epC1 : a.epC2;
        long long cnt = 0;
        filter_pass(d, n, [&](long long i) { return __ldcg(list + i); }, p0 ? &ctl->ncand : &ctl->ncand2,
                    p0 ? d.cand : d.cand2, ep, scanned, cnt, p0 ? a.epA : 0u, p0 ? np0 : 0, d.psi[0], &cnt_ins);
        hub_filter(d, s, p0 ? d.hubA : d.hubN, nh, ep, p0 ? &ctl->nhubC : &ctl->nhubC2, p0 ? d.hubC : d.hubC2,
                   scanned, cnt);  // hubs: CTA-cooperative
        if (p0) {
          block_atomic_add(&ctl->st[ST_INSERTED], cnt_ins, s.red);
          block_atomic_add(&ctl->st[ST_AFFECTED], cnt + cnt_ins, s.red);
          PHASE_FLUSH(PH_F0, n + nh + np0);
        } else {
          block_atomic_add(&ctl->st[ST_EXPANDED], cnt, s.red);
          if (tid == 0) ctl->ncand = 0;  // read by every CTA before the last barrier
          PHASE_FLUSH(PH_F2, n + nh);
        }
        GRID_SYNC_STAMPED(ctl, p0 ? 201 : 203);
      }
      {  // ---- F1: commit C1 + R2 expansion marks (+ marks of the pending-since-
         //      apply vertices' neighbours, same pass) | F3: commit C2
        const int nc = ldv(p0 ? &ctl->ncand : &ctl->ncand2), nhC = ldv(p0 ? &ctl->nhubC : &ctl->nhubC2);
        const uint32_t ep = p0 ? a.epC1 : a.epC2;
        if (tid == 0) ctl->st[p0 ? ST_FILTERED_IN : ST_EXPANDED_IN] = nc + nhC;
        commit(d, s, a, nc, p0 ? d.cand : d.cand2, ep, p0, scanned, cut_acc, p0 ? np0 : 0, d.psi[0]);
        hub_commit(d, s, a, p0 ? d.hubC : d.hubC2, nhC, ep, p0, scanned, cut_acc);
        flush_acc(s, ctl->Wp, k);
        PHASE_FLUSH(p0 ? PH_F1 : PH_F3, nc + nhC + (p0 ? np0 : 0));
        GRID_SYNC_STAMPED(ctl, p0 ? 202 : 204);
      }
    }
  } else {  // sharded: the same phases as staged launches (RefineMode)
  if (mode == kModeFull || mode == kShF0) {
  if (!kSh && a.global) {  // NEXT-1: A |= partition boundary, then the ordinary refine
    boundary_mark(d, a.epA);
    PHASE_FLUSH(PH_BOUNDARY, ldv(&ctl->n_total));
    GRID_SYNC_STAMPED(ctl, 220);
  }
  // ---- F0: pending set joins F; R1 filter over A on sigma1 -----------------
  const int nA = ldv(&ctl->nA);
  const int np0 = ldv(&ctl->npsi[0]);
  const int nhA = ldv(&ctl->nhubA);
  // R1 filter over A; the pending-since-apply vertices (psi[0]) are counted
  // in the same pass (stat `inserted`)
  filter_pass(d, nA, [&](long long i) { return __ldcg(d.Alist + i); }, &ctl->ncand, d.cand, a.epC1, scanned,
              counted, a.epA, np0, d.psi[0], &cnt_ins);  // hubs of A: CTA-cooperative below
  hub_filter(d, s, d.hubA, nhA, a.epC1, &ctl->nhubC, d.hubC, scanned, counted);
  if (kSh && d.rank != 0) cnt_ins = 0;  // replicated count: summed over the ranks, so rank 0 adds it
  block_atomic_add(&ctl->st[ST_INSERTED], cnt_ins, s.red);
  block_atomic_add(&ctl->st[ST_AFFECTED], counted + cnt_ins, s.red);
  PHASE_FLUSH(PH_F0, nA + nhA + np0);
  if (kSh) {  // this rank's C1 -> the bitmap (all-reduced by the host)
    grid.sync();
    sh_publish(d, ldv(&ctl->ncand), d.cand, ldv(&ctl->nhubC), d.hubC);
    flush_partial();
    return false;
  }
  GRID_SYNC_STAMPED(ctl, 201);
  }

  // ---- F1: commit C1 + R2 expansion marks -----------------------------------
  if (mode == kModeFull || mode == kShF1) {
  if (kSh) {  // C1 = every rank's candidates (all-reduced bitmap)
    if (tid == 0) {
      ctl->ncand = 0;
      ctl->nhubC = 0;
    }
    grid.sync();
    sh_extract(d, nwords, a.epC1, &ctl->ncand, d.cand, &ctl->nhubC, d.hubC);
    grid.sync();
    sh_clear_bm(d, nwords);
  }
  {
    const int np0 = ldv(&ctl->npsi[0]);  // pending since apply (C1 joins beyond)
    const int nc = ldv(&ctl->ncand), nhC = ldv(&ctl->nhubC);
    if (tid == 0) ctl->st[ST_FILTERED_IN] = nc + nhC;
    // commit C1 and, in the same pass, mark the neighbours of the pseudo
    // vertices pending since apply (psi[0][0, np0); C1 joins beyond np0)
    commit(d, s, a, nc, d.cand, a.epC1, true, scanned, cut_acc, np0, d.psi[0]);
    hub_commit(d, s, a, d.hubC, nhC, a.epC1, true, scanned, cut_acc);
    flush_acc(s, ctl->Wp, k);
    PHASE_FLUSH(PH_F1, nc + nhC + np0);
  }
  GRID_SYNC_STAMPED(ctl, 202);

  // ---- F2: R2 filter on sigma2 ------------------------------------------------
  {
    const int nN = ldv(&ctl->nN), nhN = ldv(&ctl->nhubN);
    long long cntN = 0;
    filter_pass(d, nN, [&](long long i) { return __ldcg(d.Nlist + i); }, &ctl->ncand2, d.cand2, a.epC2, scanned,
                cntN);
    hub_filter(d, s, d.hubN, nhN, a.epC2, &ctl->nhubC2, d.hubC2, scanned, cntN);
    block_atomic_add(&ctl->st[ST_EXPANDED], cntN, s.red);
    if (tid == 0) ctl->ncand = 0;  // read by every CTA before the last barrier
    PHASE_FLUSH(PH_F2, nN + nhN);
  }
  if (kSh) {  // this rank's C2 -> the bitmap
    grid.sync();
    sh_publish(d, ldv(&ctl->ncand2), d.cand2, ldv(&ctl->nhubC2), d.hubC2);
    flush_partial();
    return false;
  }
  GRID_SYNC_STAMPED(ctl, 203);
  }

  // ---- F3: commit C2 --------------------------------------------------------------
  if (mode == kModeFull || mode == kShF3) {
  if (kSh) {  // C2 = every rank's candidates
    if (tid == 0) {
      ctl->ncand2 = 0;
      ctl->nhubC2 = 0;
    }
    grid.sync();
    sh_extract(d, nwords, a.epC2, &ctl->ncand2, d.cand2, &ctl->nhubC2, d.hubC2);
    grid.sync();
    sh_clear_bm(d, nwords);
  }
  {
    const int nc = ldv(&ctl->ncand2), nhC2 = ldv(&ctl->nhubC2);
    if (tid == 0) ctl->st[ST_EXPANDED_IN] = nc + nhC2;
    commit(d, s, a, nc, d.cand2, a.epC2, false, scanned, cut_acc);
    hub_commit(d, s, a, d.hubC2, nhC2, a.epC2, false, scanned, cut_acc);
    flush_acc(s, ctl->Wp, k);
    PHASE_FLUSH(PH_F3, nc + nhC2);
  }
  GRID_SYNC_STAMPED(ctl, 204);
  }  // F3 (sharded)
  }  // sharded F0-F3

  // ---- R3: balance restoration (reading Q9), helpers above -------------------------
  if (mode == kModeFull || mode == kShF3) {
    const bool any = r3_setup();
    if (kSh && tid == 0) ctl->sh_flag = any;
    if (any) {
      if (tid == 0) path_hit(ctl, PA_R3);
      const long long ntot = ldv(&ctl->n_total);
      if (kSh) {  // only owners know a key: 0 everywhere else (the host all-reduces the array)
        rr_for(ntot, [&](long long v) {
          const uint8_t p = ld_part(d.part, v);
          if (p == kDel || p == kPsi || !s.sel.used[p] || !own(d, v)) d.lossbuf[v] = 0;
        });
      }
      auto emit = [&](int v, uint8_t p, long long loss) {
        if (kSh) d.lossbuf[v] = (uint32_t)(loss + 0x80000000ll);  // |loss| < 2^31 (limits: 255 * 2^23)
        else r3_emit(v, p, loss);
      };

      // keys (int - ext, id) of every vertex of an overweight part on sigma3
      auto get = [&](long long v) {
        uint8_t p = ld_part(d.part, v);
        return (p != kDel && p != kPsi && s.sel.used[p] && own(d, v)) ? (int)v : -1;
      };
      auto pre = [&](int v, long long) -> int { return ld_part(d.part, v); };  // an L1/L2 hit: get read it
      auto tf = [&](int v, long long, long long o, int dg, int pvv) {
        const uint8_t pv = (uint8_t)pvv;
        long long in = 0, ex = 0;
        nbrs_thread(d, o, dg, [&](int, int w, uint8_t q) {
          if (q == pv) in += w; else ex += w;
          return true;
        });
        scanned += dg;
        emit(v, pv, in - ex);
      };
      auto wf = [&](int v, long long, long long o, int dg, int pvv) {
        const uint8_t pv = (uint8_t)pvv;
        long long in = 0, ex = 0;
        nbrs_warp(d, o, dg, [&](int, int w, uint8_t q) {
          if (q == pv) in += w; else ex += w;
        });
        in = warp_sum(in);
        ex = warp_sum(ex);
        if (lane_id() == 0) {
          scanned += dg;
          emit(v, pv, in - ex);
        }
      };
      foreach_vertex(d, ntot, get, pre, tf, wf);
      PHASE_FLUSH(PH_R3, ntot);
      if (!kSh) {
        GRID_SYNC_STAMPED(ctl, 205);
        r3_select_evict_commit();
      }
    }
    if (kSh) {
      if (tid == 0) ctl->sh_np = ldv(&ctl->npsi[0]);  // every commit is behind barrier 204
      flush_partial();
      return false;
    }
  }
  if (kSh && mode == kShR3) {  // every rank: the all-reduced keys -> the replicated select + commit
    r3_setup();
    const long long ntot = ldv(&ctl->n_total);
    rr_for(ntot, [&](long long v) {
      const uint32_t e = __ldcg(d.lossbuf + v);
      if (e) r3_emit((int)v, ld_part(d.part, v), (long long)e - 0x80000000ll);
    });
    GRID_SYNC_STAMPED(ctl, 205);
    r3_select_evict_commit();
    if (tid == 0) ctl->sh_np = ldv(&ctl->npsi[0]);  // the eviction commit is behind barrier 207
    flush_partial();
    return false;
  }

  // ---- R4: rounds (Alg. 4), grid-wide (a CTA-local variant for small tails
  //      measured slower: the rounds are load-latency bound, not barrier bound)
  RoundState rs;
  if (kSh && sh.mode == kShPost) {
    rs.rounds = ldv(&ctl->rs_rounds);
    rs.applied_tot = ldv(&ctl->rs_applied);
    rs.deferred_tot = ldv(&ctl->rs_deferred);
  } else {
    run_rounds<kSh>(d, a, s, grid, c, exact_shift_id, rs, scanned, cut_acc, sh, pw_);
  }
  const long long rounds = rs.rounds, applied_tot = rs.applied_tot, deferred_tot = rs.deferred_tot;

  // delta list for the caller (igk_partition_delta): every vertex of the
  // frontier F (it holds all that can have moved, I4) whose label now
  // differs from its label before the refine; inserted vertices (oldp = psi)
  // are listed with their first placement.  The labels are final after the
  // last round's barrier.
  rr_for(ldv(&ctl->npsi[0]), [&](long long i) {
    const int u = __ldcg(d.psi[0] + i);
    const uint8_t p = u >= 0 ? ld_part(d.part, u) : kDel;
    const bool ch = p != kDel && p != kPsi && p != __ldcg(d.oldp + u);
    const int slot = agg_append(&ctl->n_delta, ch);
    if (ch) d.delta[slot] = make_int2(u, (int)p);
  });

  block_atomic_add(&ctl->cut, cut_acc, s.red);
  block_atomic_add(&ctl->st[ST_SCANNED], scanned, s.red);
  // no grid barrier: the LAST CTA past this point (every CTA's atomics and
  // delta entries are fenced before its arrival) finalises the stats and
  // posts the completion notice -- one grid-wide wait less per step
  __shared__ int s_fin;
  arrive_stamp(d.dbg, 11);
  if (threadIdx.x == 0) {
    __threadfence();
    s_fin = atomicAdd(&ctl->ndone_ref, 1) == (int)gridDim.x - 1;
  }
  __syncthreads();
  if (!s_fin) return true;
  if (threadIdx.x == 0) {
    __threadfence();
    ctl->ndone_ref = 0;
    const int ip = ctl->nph;  // the epilogue's phase stamp (CTA 0 wrote its earlier ones before arriving)
    if (ip < 128) {
      ctl->tph[ip] = gtimer();
      ctl->idph[ip] = 211;
      ctl->nph = ip + 1;
    }
    // every word read first (one round trip: no store in between to order
    // them behind), then the stores
    long long v[ST_N];
#pragma unroll
    for (int i = 0; i < ST_N; i++) v[i] = __ldcg(&ctl->st[i]);
    const long long cut_now = __ldcg(&ctl->cut);
    long long mx = 0;
#pragma unroll 8
    for (int p = 0; p < k; p++) mx = max(mx, __ldcg(&ctl->Wp[p]));
    v[ST_ROUNDS] = rounds;
    v[ST_MOVES_APPLIED] = applied_tot;
    v[ST_MOVES_DEFERRED] = deferred_tot;
    v[ST_CUT] = cut_now;
    v[ST_CAP] = c;
    v[ST_MAXW] = mx;
#pragma unroll
    for (int i = 0; i < ST_N; i++) {
      ctl->st_out[i] = v[i];
      ctl->st[i] = 0;
    }
    for (int r = 0; r < 3; r++) {
      ctl->applied3[r] = 0;
      ctl->selected3[r] = 0;
      for (int p = 0; p < k; p++) ctl->tot3[r][p] = 0;
    }
    ctl->nA = 0;
    ctl->nhubA = 0;
    ctl->nhubC = 0;
    ctl->nhubN = 0;
    ctl->nhubC2 = 0;
    ctl->nhubP = 0;
    ctl->ncand = 0;
    ctl->ncand2 = 0;
    ctl->nN = 0;
    ctl->nr3 = 0;
    ctl->npsi[0] = 0;
    ctl->npsi[1] = 0;
    ctl->npsi[2] = 0;
  }
  __syncthreads();
  if (!kSh) publish_copy(d);
  return true;
}

#ifndef IGK_REFINE_MINB
#define IGK_REFINE_MINB 1
#endif
__global__ void __launch_bounds__(kThreads, IGK_REFINE_MINB) k_refine(Dev d, RefineArgs a) {
  cg::grid_group grid = cg::this_grid();
  extern __shared__ __align__(16) unsigned char smem_raw[];
  ShardArgs sh{};
  sh.mode = kModeFull;
  if (!refine_body<false>(d, a, grid, *reinterpret_cast<RefSmem*>(smem_raw), sh)) publish(d);
}

// sharded refine: one launch per mode (RefineMode kSh*), driven by igk.cu refine_sharded
__global__ void __launch_bounds__(kThreads) k_refine_sh(Dev d, RefineArgs a, ShardArgs sh) {
  cg::grid_group grid = cg::this_grid();
  extern __shared__ __align__(16) unsigned char smem_raw[];
  refine_body<true>(d, a, grid, *reinterpret_cast<RefSmem*>(smem_raw), sh);
}

// ---------------------------------------------------------------------------
// NEXT-3: all rounds of a sharded refine in ONE persistent kernel per rank.
// Each round the owners store the move records of their selected vertices
// (16 B each) directly into the round's record buffer of EVERY rank (peer
// memory: NVLink P2P across GPUs, plain device memory for ranks sharing a
// GPU), then the ranks meet at a device-side barrier (system-scope atomics
// on every rank's counter, release / acquire fences) instead of a host
// round trip + all-reduce; every rank then installs all records, takes the
// same balanced prefix and applies it (the kShGain / kShFinish
// logic of run_rounds).  Two buffers alternate by round parity: a rank that
// zeroed its buffer after installing round r can only receive round r+2's
// records after everyone passed round r+1's barrier.  A peer that never
// arrives (bounded spin) sets Ctl::p2p_err and every rank stops.
// ---------------------------------------------------------------------------
struct P2PArgs {
  int n, self;                      // ranks, this rank
  int4* bufs[8][2];                 // every rank's two record buffers (by round parity)
  unsigned long long* bars[8];      // every rank's barrier counter
  unsigned long long bar_base;      // counter value before this refine's first round (n x rounds so far)
  long long timeout;                // clock64 cycles a rank waits at the barrier before giving up
};

__global__ void __launch_bounds__(kThreads) k_rounds_p2p(Dev d, RefineArgs a, long long np, P2PArgs pa) {
  cg::grid_group grid = cg::this_grid();
  extern __shared__ __align__(16) unsigned char smem_raw[];
  RefSmem& s = *reinterpret_cast<RefSmem*>(smem_raw);
  Ctl* ctl = d.ctl;
  const int k = d.k;
  const long long c = cap_of(ldv(&ctl->W), a.e_ppm, k);
  const int exact_shift_id = ((d.idbits + 7) / 8) * 8 - 8;
  for (int p = threadIdx.x; p < 256; p += blockDim.x) {
    s.acc[p] = 0;
    s.sel.used[p] = 0;
    s.sel.active[p] = 0;
  }
  for (int t = threadIdx.x; t < kWarps * 256; t += blockDim.x) (&s.wconn[0][0])[t] = 0;
  __syncthreads();
  long long scanned = 0, cut_acc = 0;
  PhaseWork pw_;
  RoundState rs;
  rs.cur = 1;
  rs.rounds = ldv(&ctl->rs_rounds);
  rs.rounds_all = ldv(&ctl->rs_rounds_all);
  rs.applied_tot = ldv(&ctl->rs_applied);
  rs.deferred_tot = ldv(&ctl->rs_deferred);
  ShardArgs sh{};
  sh.np = np;
  for (long long r = 0;; r++) {
    const int par = (int)(r & 1);
    Dev dr = d;
    dr.recs = pa.bufs[pa.self][par];  // installed from here
    dr.p2p_n = pa.n;
    for (int q = 0; q < pa.n; q++) dr.p2p_recs[q] = pa.bufs[q][par];
    sh.mode = kShGain;
    run_rounds<true>(dr, a, s, grid, c, exact_shift_id, rs, scanned, cut_acc, sh, pw_);
    __threadfence_system();  // this rank's record stores before its arrival
    grid.sync();
    if (blockIdx.x == 0 && threadIdx.x == 0) {
      for (int q = 0; q < pa.n; q++) atomicAdd_system(pa.bars[q], 1ull);
      const unsigned long long target = pa.bar_base + (unsigned long long)pa.n * (unsigned long long)(r + 1);
      const long long t0 = clock64();
      int err = 0;
      while (*(volatile unsigned long long*)pa.bars[pa.self] < target)
        if (clock64() - t0 > pa.timeout) {
          err = 1;
          break;
        }
      __threadfence_system();  // the peers' records are visible before anyone installs
      ctl->p2p_err = err;
    }
    grid.sync();
    if (ldv(&ctl->p2p_err)) break;  // uniform
    sh.mode = kShFinish;
    run_rounds<true>(dr, a, s, grid, c, exact_shift_id, rs, scanned, cut_acc, sh, pw_);
    rr_for(np, [&](long long j) { dr.recs[j] = make_int4(0, 0, 0, 0); });  // free for round r + 2
    grid.sync();
    if (ldv(&ctl->rs_pending) == 0) break;
  }
  block_atomic_add(&ctl->cut, cut_acc, s.red);
  block_atomic_add(&ctl->st[ST_SCANNED], scanned, s.red);
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    ctl->rs_rounds = rs.rounds;
    ctl->rs_rounds_all = rs.rounds_all;
    ctl->rs_applied = rs.applied_tot;
    ctl->rs_deferred = rs.deferred_tot;
  }
}

}  // namespace igk
