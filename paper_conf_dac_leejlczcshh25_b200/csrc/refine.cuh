// refine.cuh -- incremental refinement (Sec. V.C) as one persistent kernel.
//
//   R1 filter over the affected set A          (Alg. 3 L8-24)
//   deferred commit to the pseudo-partition    (Alg. 3 L25-26)
//   R2 expansion: neighbours of pseudo vertices, filter, commit
//   R3 balance restoration (paper silent; reading Q9): evict the minimum-loss
//      vertices of every overweight part by a weighted device radix select
//   R4 rounds (Alg. 4) until the pseudo-partition is empty:
//      select (no smaller-ID pseudo neighbour) + best part (one adjacency
//      pass, O(deg + k)) | balanced prefix by weighted radix select of the
//      first violating move in (#nbr desc, ID asc) order | apply.
// The paper's sort + k*M segmented scan is replaced by a select
// that finds the same prefix length without sorting.
#pragma once
#include "common.cuh"

namespace igk {

struct RefineArgs {
  long long e_ppm;
  uint32_t epC1, epN, epC2, epE;
};

// ---------------------------------------------------------------------------
// per-vertex scans
// ---------------------------------------------------------------------------
// internal / external weighted degree on the current partition (
// pseudo neighbours are external, Q13).  Thread variant.
__device__ __forceinline__ void int_ext_thread(const Dev& d, int u, uint8_t pu, long long& in,
                                               long long& ex) {
  const long long o = __ldg(d.off + u);
  const int dg = __ldg(d.deg + u);
  long long a = 0, b = 0;
  for (int i = 0; i < dg; i++) {
    int x = __ldg(d.adj + o + i);
    int w = edge_w(d.adjw, o + i);
    if (ld_part(d.part, x) == pu) a += w; else b += w;
  }
  in = a;
  ex = b;
}
// warp variant (all lanes get the totals)
__device__ __forceinline__ void int_ext_warp(const Dev& d, int u, uint8_t pu, long long& in,
                                             long long& ex) {
  const long long o = __ldg(d.off + u);
  const int dg = __ldg(d.deg + u);
  long long a = 0, b = 0;
  for (int i = lane_id(); i < dg; i += 32) {
    int x = __ldg(d.adj + o + i);
    int w = edge_w(d.adjw, o + i);
    if (ld_part(d.part, x) == pu) a += w; else b += w;
  }
  in = warp_sum(a);
  ex = warp_sum(b);
}

// Iterate a vertex list: degree <= kThreadDeg -> one thread, else the whole
// warp cooperates on it.  get(i) -> vertex (or -1); tf(u, i); wf(u, i).
template <class Get, class TF, class WF>
__device__ __forceinline__ void foreach_vertex(const Dev& d, long long n, Get get, TF tf, WF wf) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (long long base = (long long)blockIdx.x * blockDim.x + (threadIdx.x & ~31); base < n; base += stride) {
    long long i = base + lane_id();
    int u = i < n ? get(i) : -1;
    int dg = u >= 0 ? __ldg(d.deg + u) : 0;
    bool heavy = dg > kThreadDeg;
    if (u >= 0 && !heavy) tf(u, i);
    unsigned hm = __ballot_sync(0xffffffffu, heavy);
    while (hm) {
      int src = __ffs(hm) - 1;
      hm &= hm - 1;
      int uu = __shfl_sync(0xffffffffu, u, src);
      wf(uu, base + src);
    }
  }
}

// ---------------------------------------------------------------------------
// weighted radix select (shared by R3 and the round prefix)
// Per candidate part p: find the first item, in ascending key order among the
// items of part p, whose inclusive weight prefix reaches T_p.  Key =
// (d0, R): d0 is an 8-bit digit built in the producing phase; R is the item's
// vertex ID when bin d0 is exact, else a full 64-bit key.  MSD passes of 8
// bits over R, one grid barrier per pass; every CTA recomputes the digit
// choice from the global histograms, so no extra barrier is needed.
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

// digit-0 choice for every candidate part (cands: flags per part in sm.used)
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

// accumulate pass `pass` histograms; items(j, &p, &d0, &R, &w) -> valid
template <class Items>
__device__ void sel_accumulate(const Dev& d, SelSmem& sm, int pass, long long nitems, Items items) {
  long long* hb = d.histR + (long long)(pass % 3) * 256 * kDigits;
  long long* hz = d.histR + (long long)((pass + 1) % 3) * 256 * kDigits;
  const long long tid = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  const long long nthr = (long long)gridDim.x * blockDim.x;
  for (long long t = tid; t < (long long)d.k * kDigits; t += nthr)
    if (sm.active[t / kDigits]) hz[t] = 0;
  for (long long j = tid; j < nitems; j += nthr) {
    int p, d0;
    unsigned long long R;
    long long w;
    if (!items(j, p, d0, R, w)) continue;
    if (!sm.active[p] || d0 != sm.d0[p]) continue;
    int sh = sm.shift[p];
    if (sh + 8 < 64 && (R >> (sh + 8)) != (sm.prefix[p] >> (sh + 8))) continue;
    int dig = (int)((R >> sh) & 255);
    atomic_add_ll(hb + (long long)p * kDigits + dig, w);
  }
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

// full select: digit 0 from d.hist0, then passes; returns after the last pass
template <class ExactFn, class Items>
__device__ void weighted_select(const Dev& d, SelSmem& sm, cg::grid_group& grid, ExactFn is_exact,
                                int exact_shift, long long nitems, Items items) {
  sel_digit0(d, sm, is_exact, exact_shift);
  int pass = 0;
  while (sm.nactive > 0) {
    sel_accumulate(d, sm, pass, nitems, items);
    grid.sync();
    sel_choose(d, sm, pass);
    pass++;
  }
  // every CTA must finish reading the histograms before anyone clears them
  if (pass > 0) grid.sync();
}

// zero the histogram rows the select used (call after every CTA finished it)
__device__ void sel_clear(const Dev& d, const SelSmem& sm) {
  const long long tid = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  const long long nthr = (long long)gridDim.x * blockDim.x;
  for (long long t = tid; t < (long long)d.k * kDigits; t += nthr) {
    if (!sm.used[t / kDigits]) continue;
    d.hist0[t] = 0;
    d.histR[t] = 0;
    d.histR[256 * kDigits + t] = 0;
    d.histR[2 * 256 * kDigits + t] = 0;
  }
}

// ---------------------------------------------------------------------------
// the refine kernel
// ---------------------------------------------------------------------------
struct RefSmem {
  SelSmem sel;
  long long Wr[256];      // round-start part weights (Q14)
  long long acc[256];     // per-part weight deltas of this CTA
  long long red[32];
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

// candidate-set commit (Alg. 3 L25-26): cut and W_p deltas on the snapshot
// before any label changes; edges between two candidates counted once.
__device__ void commit_delta(const Dev& d, RefSmem& s, int nc, uint32_t ep, long long& cut_acc) {
  auto get = [&](long long i) { return __ldcg(d.cand + i); };
  auto delta_thread = [&](int u, long long) {
    const uint8_t pu = ld_part(d.part, u);
    const long long o = __ldg(d.off + u);
    const int dg = __ldg(d.deg + u);
    long long del = 0;
    for (int i = 0; i < dg; i++) {
      int x = __ldg(d.adj + o + i);
      uint8_t px = ld_part(d.part, x);
      if (px != kPsi && px != pu && !(x < u && __ldcg(d.markT + x) == ep)) del += edge_w(d.adjw, o + i);
    }
    cut_acc -= del;
    atomicAdd((unsigned long long*)&s.acc[pu], (unsigned long long)(-(long long)vert_w(d.vw, u)));
  };
  auto delta_warp = [&](int u, long long) {
    const uint8_t pu = ld_part(d.part, u);
    const long long o = __ldg(d.off + u);
    const int dg = __ldg(d.deg + u);
    long long del = 0;
    for (int i = lane_id(); i < dg; i += 32) {
      int x = __ldg(d.adj + o + i);
      uint8_t px = ld_part(d.part, x);
      if (px != kPsi && px != pu && !(x < u && __ldcg(d.markT + x) == ep)) del += edge_w(d.adjw, o + i);
    }
    del = warp_sum(del);
    if (lane_id() == 0) {
      cut_acc -= del;
      atomicAdd((unsigned long long*)&s.acc[pu], (unsigned long long)(-(long long)vert_w(d.vw, u)));
    }
  };
  foreach_vertex(d, nc, get, delta_thread, delta_warp);
}

__device__ void commit_write(const Dev& d, int nc, int* psi_cnt, int32_t* psi_list) {
  const long long tid = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  const long long nthr = (long long)gridDim.x * blockDim.x;
  for (long long i = tid; i < nc; i += nthr) {
    int u = __ldcg(d.cand + i);
    d.part[u] = kPsi;
    int slot = agg_append(psi_cnt, true);
    psi_list[slot] = u;
  }
}

// filter (Alg. 3 L8-24): candidates = listed placed vertices with ext > int
template <class Get>
__device__ void filter_pass(const Dev& d, long long n, Get get, uint32_t ep, long long& scanned,
                            long long& counted) {
  Ctl* ctl = d.ctl;
  auto tf = [&](int u, long long) {
    if (!__ldcg(d.active + u)) return;
    uint8_t pu = ld_part(d.part, u);
    if (pu == kPsi) return;
    counted++;
    long long in, ex;
    int_ext_thread(d, u, pu, in, ex);
    scanned += __ldg(d.deg + u);
    bool c = ex > in;
    if (c) {
      d.markT[u] = ep;
      int slot = atomicAdd(&ctl->ncand, 1);
      d.cand[slot] = u;
    }
  };
  auto wf = [&](int u, long long) {
    if (!__ldcg(d.active + u)) return;
    uint8_t pu = ld_part(d.part, u);
    if (pu == kPsi) return;
    long long in, ex;
    int_ext_warp(d, u, pu, in, ex);
    if (lane_id() == 0) {
      counted++;
      scanned += __ldg(d.deg + u);
      if (ex > in) {
        d.markT[u] = ep;
        int slot = atomicAdd(&ctl->ncand, 1);
        d.cand[slot] = u;
      }
    }
  };
  foreach_vertex(d, n, get, tf, wf);
}

// better(a, b) on (conn desc, W_p asc, p asc)  (reading Q6)
__device__ __forceinline__ bool better(long long ca, int pa, long long cb, int pb, const long long* Wr) {
  if (pb < 0) return true;
  if (ca != cb) return ca > cb;
  if (Wr[pa] != Wr[pb]) return Wr[pa] < Wr[pb];
  return pa < pb;
}

__global__ void __launch_bounds__(kThreads) k_refine(Dev d, RefineArgs a) {
  cg::grid_group grid = cg::this_grid();
  extern __shared__ __align__(16) unsigned char smem_raw[];
  RefSmem& s = *reinterpret_cast<RefSmem*>(smem_raw);
  Ctl* ctl = d.ctl;
  const int k = d.k;
  const long long tid = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  const long long nthr = (long long)gridDim.x * blockDim.x;
  const long long c = cap_of(ldv(&ctl->W), a.e_ppm, k);
  const int exact_shift_id = ((d.idbits + 7) / 8) * 8 - 8;

  for (int p = threadIdx.x; p < 256; p += blockDim.x) {
    s.acc[p] = 0;
    s.sel.used[p] = 0;
    s.sel.active[p] = 0;
  }
  for (int t = threadIdx.x; t < kWarps * 256; t += blockDim.x) (&s.wconn[0][0])[t] = 0;
  __syncthreads();

  long long cut_acc = 0, scanned = 0, counted = 0, cnt_ins = 0;
  // ---- F0: stats of the pending set; R1 filter over A on sigma1 -------------
  const int nA = ldv(&ctl->nA);
  const int np0 = ldv(&ctl->npsi[0]);
  for (long long i = tid; i < np0; i += nthr) {
    int u = __ldcg(d.psi[0] + i);
    if (__ldcg(d.active + u) && ld_part(d.part, u) == kPsi) cnt_ins++;
  }
  filter_pass(d, nA, [&](long long i) { return __ldcg(d.Alist + i); }, a.epC1, scanned, counted);
  block_atomic_add(&ctl->st[ST_INSERTED], cnt_ins, s.red);
  block_atomic_add(&ctl->st[ST_AFFECTED], counted + cnt_ins, s.red);
  grid.sync();

  // ---- F1/F2: commit C1 -------------------------------------------------------
  int nc = ldv(&ctl->ncand);
  commit_delta(d, s, nc, a.epC1, cut_acc);
  flush_acc(s, ctl->Wp, k);
  grid.sync();
  commit_write(d, nc, &ctl->npsi[0], d.psi[0]);
  if (tid == 0) ctl->st[ST_FILTERED_IN] = nc;
  grid.sync();

  // ---- F3: R2 expansion: placed neighbours of every pseudo vertex ---
  {
    const int np = ldv(&ctl->npsi[0]);
    if (tid == 0) ctl->ncand = 0;
    auto get = [&](long long i) {
      int u = __ldcg(d.psi[0] + i);
      return (__ldcg(d.active + u) && ld_part(d.part, u) == kPsi) ? u : -1;
    };
    auto tf = [&](int u, long long) {
      const long long o = __ldg(d.off + u);
      const int dg = __ldg(d.deg + u);
      scanned += dg;
      for (int i = 0; i < dg; i++) {
        int x = __ldg(d.adj + o + i);
        if (ld_part(d.part, x) != kPsi && stamp_insert(d.markT, x, a.epN))
          d.Nlist[atomicAdd(&ctl->nN, 1)] = x;
      }
    };
    auto wf = [&](int u, long long) {
      const long long o = __ldg(d.off + u);
      const int dg = __ldg(d.deg + u);
      if (lane_id() == 0) scanned += dg;
      for (int i = lane_id(); i < dg; i += 32) {
        int x = __ldg(d.adj + o + i);
        bool add = ld_part(d.part, x) != kPsi && stamp_insert(d.markT, x, a.epN);
        int slot = agg_append(&ctl->nN, add);
        if (add) d.Nlist[slot] = x;
      }
    };
    foreach_vertex(d, np, get, tf, wf);
  }
  grid.sync();

  // ---- F4: R2 filter on sigma2 ---------------------------------------------
  {
    const int nN = ldv(&ctl->nN);
    long long dummy = 0;
    filter_pass(d, nN, [&](long long i) { return __ldcg(d.Nlist + i); }, a.epC2, scanned, dummy);
    if (tid == 0) ctl->st[ST_EXPANDED] = nN;
  }
  grid.sync();
  nc = ldv(&ctl->ncand);
  commit_delta(d, s, nc, a.epC2, cut_acc);
  flush_acc(s, ctl->Wp, k);
  grid.sync();
  commit_write(d, nc, &ctl->npsi[0], d.psi[0]);
  if (tid == 0) ctl->st[ST_EXPANDED_IN] = nc;
  grid.sync();

  // ---- R3: balance restoration (reading Q9) -----------------------------------
  {
    bool any = false;
    for (int p = 0; p < k; p++) any |= ldv(&ctl->Wp[p]) > c;
    if (any) {
      if (tid == 0) ctl->ncand = 0;
      for (int p = threadIdx.x; p < k; p += blockDim.x) {
        long long wp = ldv(&ctl->Wp[p]);
        s.sel.used[p] = wp > c;
        s.sel.T[p] = wp - c;
      }
      __syncthreads();
      // keys (int - ext, id) for every vertex of an overweight part, sigma3
      const long long ntot = ldv(&ctl->n_total);
      auto get = [&](long long v) {
        if (!__ldcg(d.active + v)) return -1;
        uint8_t p = ld_part(d.part, v);
        return (p != kPsi && s.sel.used[p]) ? (int)v : -1;
      };
      auto emit = [&](int v, long long loss) {
        uint8_t p = ld_part(d.part, v);
        int d0 = (int)max(0ll, min(255ll, loss + 128));
        atomic_add_ll(d.hist0 + (long long)p * kDigits + d0, vert_w(d.vw, v));
        int slot = atomicAdd(&ctl->nr3, 1);
        d.r3list[slot] = make_int2(v, (int)loss);
      };
      auto tf = [&](int v, long long) {
        long long in, ex;
        int_ext_thread(d, v, ld_part(d.part, v), in, ex);
        scanned += __ldg(d.deg + v);
        emit(v, in - ex);
      };
      auto wf = [&](int v, long long) {
        long long in, ex;
        int_ext_warp(d, v, ld_part(d.part, v), in, ex);
        if (lane_id() == 0) {
          scanned += __ldg(d.deg + v);
          emit(v, in - ex);
        }
      };
      foreach_vertex(d, ntot, get, tf, wf);
      grid.sync();
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
      // evict every item with key <= the threshold of its part
      for (long long j = tid; j < nr3; j += nthr) {
        int p, d0;
        unsigned long long R;
        long long w;
        items(j, p, d0, R, w);
        if (!s.sel.found[p]) continue;
        if (!key_less(s.sel.d0[p], s.sel.prefix[p], d0, R)) {
          int v = __ldcg(d.r3list + j).x;
          d.markT[v] = a.epE;
          d.cand[atomicAdd(&ctl->ncand, 1)] = v;
        }
      }
      sel_clear(d, s.sel);
      grid.sync();
      nc = ldv(&ctl->ncand);
      commit_delta(d, s, nc, a.epE, cut_acc);
      flush_acc(s, ctl->Wp, k);
      grid.sync();
      commit_write(d, nc, &ctl->npsi[0], d.psi[0]);
      if (tid == 0) {
        ctl->st[ST_EVICTED] = nc;
        ctl->nr3 = 0;
      }
      for (int p = threadIdx.x; p < 256; p += blockDim.x) s.sel.used[p] = 0;
      grid.sync();
    }
  }

  // ---- R4: rounds (Alg. 4) ------------------------------------------------------
  int cur = 0;
  long long rounds = 0, rounds_all = 0, applied_tot = 0, deferred_tot = 0;
  while (true) {
    const int np = ldv(&ctl->npsi[cur]);
    if (np == 0) break;
    int32_t* plist = d.psi[cur];
    int32_t* pnext = d.psi[cur ^ 1];
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
    const int r3 = (int)(rounds_all % 3), r3n = (int)((rounds_all + 1) % 3);
    if (tid == 0) {
      ctl->npsi[cur ^ 1] = 0;
      ctl->applied3[r3n] = 0;
      ctl->selected3[r3n] = 0;
    }
    for (int p = (int)tid; p < k; p += (int)nthr) ctl->tot3[r3n][p] = 0;
    // -- gain: selection + best part, one adjacency pass per vertex
    long long sel_cnt = 0;
    auto emit_move = [&](long long j, int u, int best, long long g, long long pwv, bool imbal) {
      int d0 = 255 - (int)min(g, 255ll);
      d.tgt[u] = (uint8_t)best;
      d.gain[u] = (int)g;
      d.pw[u] = (int)pwv;
      d.meta[j] = 0x80000000u | ((unsigned)d0 << 8) | (unsigned)best;
      long long w = vert_w(d.vw, u);
      atomic_add_ll(d.hist0 + (long long)best * kDigits + d0, w);
      atomic_add_ll(&ctl->tot3[r3][best], w);
      if (imbal) ctl->st[ST_IMBAL] = 1;
    };
    auto get = [&](long long i) {
      int u = __ldcg(plist + i);
      if (u < 0 || !__ldcg(d.active + u) || ld_part(d.part, u) != kPsi) {
        d.meta[i] = 0;
        return -1;
      }
      return u;
    };
    auto tf = [&](int u, long long j) {
      const long long o = __ldg(d.off + u);
      const int dg = __ldg(d.deg + u);
      const long long vwu = vert_w(d.vw, u);
      scanned += dg;
      int qs[kThreadDeg];
      int ws[kThreadDeg];
      int m = 0;
      long long pwv = 0;
      bool sel = true;
      for (int i = 0; i < dg; i++) {
        int x = __ldg(d.adj + o + i);
        uint8_t q = ld_part(d.part, x);
        if (q == kPsi) {
          if (x < u) { sel = false; break; }
          continue;
        }
        int w = edge_w(d.adjw, o + i);
        qs[m] = q;
        ws[m] = w;
        m++;
        pwv += w;
      }
      if (!sel) {
        d.meta[j] = 0;
        return;
      }
      int best = -1;
      long long bc = -1;
      for (int i = 0; i < m; i++) {
        int p = qs[i];
        bool seen = false;
        for (int t = 0; t < i; t++) seen |= qs[t] == p;
        if (seen) continue;
        long long cc = 0;
        for (int t = i; t < m; t++) cc += qs[t] == p ? ws[t] : 0;
        if (s.Wr[p] + vwu > c) continue;
        if (better(cc, p, bc, best, s.Wr)) { best = p; bc = cc; }
      }
      bool imbal = false;
      if (best < 0) {  // lightest part: eligible => zero connectivity; else fallback (Q8)
        best = s.best0;
        bc = 0;
        if (s.Wr[best] + vwu > c) {
          imbal = true;
          for (int t = 0; t < m; t++) bc += qs[t] == best ? ws[t] : 0;
        }
      }
      sel_cnt++;
      emit_move(j, u, best, bc, pwv, imbal);
    };
    auto wf = [&](int u, long long j) {
      const long long o = __ldg(d.off + u);
      const int dg = __ldg(d.deg + u);
      const long long vwu = vert_w(d.vw, u);
      int* wc = s.wconn[warp_id()];
      if (lane_id() == 0) scanned += dg;
      long long pwv = 0;
      bool blocked = false;
      for (int b = 0; b < dg && !blocked; b += 32) {
        int i = b + lane_id();
        bool lb = false;
        if (i < dg) {
          int x = __ldg(d.adj + o + i);
          uint8_t q = ld_part(d.part, x);
          if (q == kPsi) {
            lb = x < u;
          } else {
            int w = edge_w(d.adjw, o + i);
            atomicAdd(wc + q, w);
            pwv += w;
          }
        }
        blocked = __any_sync(0xffffffffu, lb);
      }
      __syncwarp();
      if (blocked) {
        for (int p = lane_id(); p < k; p += 32) wc[p] = 0;
        __syncwarp();
        if (lane_id() == 0) d.meta[j] = 0;
        return;
      }
      pwv = warp_sum(pwv);
      long long bc = -1;
      int best = -1;
      for (int p = lane_id(); p < k; p += 32) {
        if (s.Wr[p] + vwu > c) continue;
        long long cc = wc[p];
        if (better(cc, p, bc, best, s.Wr)) { best = p; bc = cc; }
      }
#pragma unroll
      for (int off = 16; off > 0; off >>= 1) {
        long long oc = __shfl_xor_sync(0xffffffffu, bc, off);
        int op = __shfl_xor_sync(0xffffffffu, best, off);
        if (op >= 0 && better(oc, op, bc, best, s.Wr)) { bc = oc; best = op; }
      }
      bool imbal = false;
      if (best < 0) {
        best = s.best0;
        bc = wc[best];
        imbal = true;
      }
      __syncwarp();
      for (int p = lane_id(); p < k; p += 32) wc[p] = 0;
      __syncwarp();
      if (lane_id() == 0) {
        sel_cnt++;
        emit_move(j, u, best, bc, pwv, imbal);
      }
    };
    foreach_vertex(d, np, get, tf, wf);
    {
      long long sc = warp_sum(sel_cnt);
      if (lane_id() == 0 && sc) atomicAdd(&ctl->selected3[r3], (int)sc);
    }
    grid.sync();

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
      if (!(m & 0x80000000u)) return false;
      int u = __ldcg(plist + j);
      p = (int)(m & 255u);
      d0 = (int)((m >> 8) & 255u);
      R = d0 ? (unsigned long long)u
             : (((unsigned long long)(0x7fffffffu - (unsigned)__ldcg(d.gain + u))) << 32) | (unsigned)u;
      w = vert_w(d.vw, u);
      return true;
    };
    weighted_select(d, s.sel, grid, [](int d0) { return d0 != 0; }, exact_shift_id, np, items);
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
    for (long long j = tid; j < np; j += nthr) {
      int u = __ldcg(plist + j);
      if (u < 0) continue;
      unsigned m = __ldcg(d.meta + j);
      bool keep = true;
      if (m & 0x80000000u) {
        int p, d0;
        unsigned long long R;
        long long w;
        items(j, p, d0, R, w);
        if (key_less(d0, R, kd, kr)) {
          keep = false;
          d.part[u] = (uint8_t)p;
          atomicAdd((unsigned long long*)&s.acc[p], (unsigned long long)w);
          cut_acc += (long long)__ldcg(d.pw + u) - __ldcg(d.gain + u);
          app++;
        }
      } else if (!__ldcg(d.active + u) || ld_part(d.part, u) != kPsi) {
        keep = false;  // stale entry (deleted before this refine)
      }
      int slot = agg_append(&ctl->npsi[cur ^ 1], keep);
      if (keep) pnext[slot] = u;
    }
    flush_acc(s, ctl->Wp, k);
    {
      long long sa = warp_sum(app);
      if (lane_id() == 0 && sa) atomicAdd(&ctl->applied3[r3], (int)sa);
    }
    // every part that received a selected move has hist0 entries: clear all rows
    for (long long t = tid; t < (long long)k * kDigits; t += nthr) d.hist0[t] = 0;
    sel_clear(d, s.sel);
    grid.sync();
    const int napp = ldv(&ctl->applied3[r3]), nsel = ldv(&ctl->selected3[r3]);
    if (napp == 0 && nsel > 0) {
      // L = 0: force the first move (reading Q8); it is the threshold item K*
      const int uf = (int)(kr & 0xffffffffu);
      const int nn = ldv(&ctl->npsi[cur ^ 1]);
      for (long long j = tid; j < nn; j += nthr)
        if (__ldcg(pnext + j) == uf) pnext[j] = -1;
      if (tid == 0) {
        int p = __ldcg(d.tgt + uf);
        d.part[uf] = (uint8_t)p;
        atomic_add_ll(&ctl->Wp[p], vert_w(d.vw, uf));
        atomic_add_ll(&ctl->cut, (long long)__ldcg(d.pw + uf) - __ldcg(d.gain + uf));
        ctl->st[ST_IMBAL] = 1;
      }
      grid.sync();
    }
    const int napp2 = napp == 0 && nsel > 0 ? 1 : napp;
    if (nsel > 0) {
      rounds++;
      applied_tot += napp2;
      deferred_tot += nsel - napp2;
    }
    for (int p = threadIdx.x; p < 256; p += blockDim.x) s.sel.used[p] = 0;
    __syncthreads();
    cur ^= 1;
    rounds_all++;
  }

  // ---- epilogue: stats and counter resets ---------------------------------------
  block_atomic_add(&ctl->cut, cut_acc, s.red);
  block_atomic_add(&ctl->st[ST_SCANNED], scanned, s.red);
  grid.sync();
  if (tid == 0) {
    ctl->st[ST_ROUNDS] = rounds;
    ctl->st[ST_MOVES_APPLIED] = applied_tot;
    ctl->st[ST_MOVES_DEFERRED] = deferred_tot;
    ctl->st[ST_CUT] = ctl->cut;
    ctl->st[ST_CAP] = c;
    long long mx = 0;
    for (int p = 0; p < k; p++) mx = max(mx, ctl->Wp[p]);
    ctl->st[ST_MAXW] = mx;
    for (int i = 0; i < ST_N; i++) {
      ctl->st_out[i] = ctl->st[i];
      ctl->st[i] = 0;
    }
    for (int r = 0; r < 3; r++) {
      ctl->applied3[r] = 0;
      ctl->selected3[r] = 0;
      for (int p = 0; p < k; p++) ctl->tot3[r][p] = 0;
    }
    ctl->nA = 0;
    ctl->ncand = 0;
    ctl->nN = 0;
    ctl->nr3 = 0;
    ctl->npsi[0] = 0;
    ctl->npsi[1] = 0;
  }
}

}  // namespace igk
