// apply.cuh -- S1: validate and apply one modifier batch on the device.
//
// One persistent cooperative kernel, four phases, three grid barriers:
//   V1  count VERTEX_INSERTs per CTA chunk, duplicate-edge hash, per-vertex counts
//   V2  validate against the pre-batch state; new IDs; slot allocation for
//       growing prefixes; 32-neighbour work chunks of every vertex deletion
//   M12 edge deletions and vertex deletions (Alg. 2, both directions,
//       reading Q12) as tombstones; marks (Alg. 3 L6-7); cut / W deltas
//   M3  finalize deletions; growing prefixes move (compacted) to new slots,
//       leaving forward marks; vertex insertions (Alg. 2 L7-10, Alg. 3 L2-5)
//   M4  edge insertions (Alg. 1) appended to the prefixes; twin fix-ups
// Every slot keeps the slot of its reverse entry ("twin"), so an edge deletion
// searches only the shorter of the two prefixes and a vertex deletion needs
// no search at all; hub prefixes (degree up to 10^4) are never scanned.
// Tombstones (-1) stay in a prefix until it relocates (lazy compaction).
// Semantics: reading S1.  Differences from the paper's design
// (DESIGN.md 5): dense-prefix adjacency with slack instead of 32-slot buckets;
// all updates of a batch are validated first and then applied as set
// operations, so concurrent updates of one vertex are race-free (Q10).
#pragma once
#include "common.cuh"

namespace igk {

struct ApplyArgs {
  const int4* mods;
  long long B;
  long long n0;  // n_total before the batch
  uint32_t epD, epT, epG, epA;
  int vw_unit, ew_unit;
  int phases;  // bit 0: V1 + V2 (validate, allocate); bit 1: M12..M4 (mutate).  Sharded handles
               // run them as two launches with the all-reduced verdict in between; else 3.
};

// Sharded store (common.cuh Dev::nranks): an edge modifier is applied on the
// ranks that own one of its endpoints (both directions are stored there);
// vertex modifiers everywhere (labels, weights, W, W_p are replicated).  The
// cut is a per-rank partial: an edge event is counted by owner(m.y), the
// edges of a deleted vertex by owner(u).
__device__ __forceinline__ bool rel_edge(const Dev& d, const int4& m) { return own(d, m.y) || own(d, m.z); }

__device__ __forceinline__ unsigned long long edge_key(int u, int v) {
  unsigned a = (unsigned)min(u, v), b = (unsigned)max(u, v);
  return ((unsigned long long)a << 32) | b;
}
__device__ __forceinline__ long long hslot(unsigned long long key, long long mask) {
  unsigned long long h = key;  // splitmix64 finalizer: every key bit reaches the low bits
  h = (h ^ (h >> 30)) * 0xBF58476D1CE4E5B9ull;
  h = (h ^ (h >> 27)) * 0x94D049BB133111EBull;
  h ^= h >> 31;
  return (long long)(h & (unsigned long long)mask);
}

// thread-level search of x in a prefix; 8 independent loads in flight
__device__ __forceinline__ long long thread_find(const int32_t* adj, long long o, int dg, int x) {
  for (int i = 0; i < dg; i += 8) {
    int v[8];
#pragma unroll
    for (int t = 0; t < 8; t++) v[t] = (i + t < dg) ? __ldcg(adj + o + i + t) : -1;
#pragma unroll
    for (int t = 0; t < 8; t++)
      if (v[t] == x) return o + i + t;
  }
  return -1;
}

// warp-cooperative search; 256 entries (8 loads per lane) per round trip
__device__ __forceinline__ long long warp_find(const int32_t* adj, long long o, int dg, int x) {
  const int lane = lane_id();
  for (int b = 0; b < dg; b += 256) {
    int v[8];
#pragma unroll
    for (int t = 0; t < 8; t++) {
      int i = b + t * 32 + lane;
      v[t] = i < dg ? __ldcg(adj + o + i) : -1;
    }
#pragma unroll
    for (int t = 0; t < 8; t++) {
      unsigned m = __ballot_sync(0xffffffffu, v[t] == x);
      if (m) return o + b + t * 32 + __ffs(m) - 1;
    }
  }
  return -1;
}

// block-wide exclusive scan of one int per thread; returns exclusive prefix, *total
__device__ __forceinline__ int block_excl_scan(int v, int* total, int* sbuf) {
  int lane = lane_id(), w = warp_id();
  int x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    int y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) sbuf[w] = x;
  __syncthreads();
  if (w == 0) {
    int t = lane < (int)(blockDim.x >> 5) ? sbuf[lane] : 0;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      int y = __shfl_up_sync(0xffffffffu, t, o);
      if (lane >= o) t += y;
    }
    sbuf[32 + lane] = t;  // inclusive over warps
  }
  __syncthreads();
  int warp_excl = w ? sbuf[32 + w - 1] : 0;
  *total = sbuf[32 + (int)(blockDim.x >> 5) - 1];
  __syncthreads();
  return warp_excl + x - v;
}

// x joins the affected set A (Alg. 3 L6-7); a vertex of degree >
// kBlockDeg is also listed (and stamped) for CTA-cooperative filtering
__device__ __forceinline__ void mark_affected(const Dev& d, int x, uint32_t epA, int dgx) {
  bool na = stamp_insert(d.markA, x, epA);
  int s2 = agg_append(&d.ctl->nA, na);
  if (na) d.Alist[s2] = x;
  if (na && dgx > kBlockDeg) {
    d.markH[x] = epA;
    d.hubA[atomicAdd(&d.ctl->nhubA, 1)] = x;
  }
}

// mark_affected with the stamp already loaded (issued with other loads)
__device__ __forceinline__ void mark_affected_pre(const Dev& d, int x, uint32_t epA, int dgx, uint32_t stamp) {
  const bool na = stamp != epA && atomicExch(d.markA + x, epA) != epA;
  int s2 = agg_append(&d.ctl->nA, na);
  if (na) d.Alist[s2] = x;
  if (na && dgx > kBlockDeg) {
    d.markH[x] = epA;
    d.hubA[atomicAdd(&d.ctl->nhubA, 1)] = x;
  }
}

// both endpoints of an edge modifier join A: stamps preloaded, both
// exchanges in flight together, one warp-aggregated list reservation
__device__ __forceinline__ void mark_affected_pair(const Dev& d, int x0, int x1, uint32_t epA, int dg0, int dg1,
                                                   uint32_t st0, uint32_t st1) {
  const bool na0 = st0 != epA && atomicExch(d.markA + x0, epA) != epA;
  const bool na1 = st1 != epA && atomicExch(d.markA + x1, epA) != epA;  // (x0 == x1: sees the first)
  int s2 = agg_alloc(&d.ctl->nA, (int)na0 + (int)na1);
  if (na0) d.Alist[s2++] = x0;
  if (na1) d.Alist[s2] = x1;
  if (na0 && dg0 > kBlockDeg) {
    d.markH[x0] = epA;
    d.hubA[atomicAdd(&d.ctl->nhubA, 1)] = x0;
  }
  if (na1 && dg1 > kBlockDeg) {
    d.markH[x1] = epA;
    d.hubA[atomicAdd(&d.ctl->nhubA, 1)] = x1;
  }
}

// mark_affected for C candidates of one thread: every stamp probe and
// exchange in flight together, one list reservation per thread
template <int C>
__device__ __forceinline__ void mark_affected_chunk(const Dev& d, const int* x, const int* dgx, const bool* want,
                                                    uint32_t epA) {
  bool w2[C];
#pragma unroll
  for (int t = 0; t < C; t++) w2[t] = want[t] && __ldcg(d.markA + x[t]) != epA;
  bool na[C];
#pragma unroll
  for (int t = 0; t < C; t++) na[t] = w2[t] && atomicExch(d.markA + x[t], epA) != epA;
  int c = 0;
#pragma unroll
  for (int t = 0; t < C; t++) c += na[t];
  if (!c) return;
  int slot = atomicAdd(&d.ctl->nA, c);
#pragma unroll
  for (int t = 0; t < C; t++) {
    if (!na[t]) continue;
    d.Alist[slot++] = x[t];
    if (dgx[t] > kBlockDeg) {
      d.markH[x[t]] = epA;
      d.hubA[atomicAdd(&d.ctl->nhubA, 1)] = x[t];
    }
  }
}

struct ApplySmem {
  int scan[64];
  long long red[32];
  long long ins[2];
};

// the whole apply; returns false (uniformly) if the batch was rejected
__device__ __forceinline__ bool apply_body(const Dev& d, const ApplyArgs& a, cg::grid_group& grid, ApplySmem& sm) {
  int* s_scan = sm.scan;
  long long* s_red = sm.red;
  Ctl* ctl = d.ctl;
  const long long tid = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  const long long nthr = (long long)gridDim.x * blockDim.x;
  const long long gwarp = tid >> 5, nwarp = nthr >> 5;
  const long long B = a.B, n0 = a.n0;
  const long long chunk = (B + gridDim.x - 1) / gridDim.x;
  const long long c_lo = min(B, (long long)blockIdx.x * chunk), c_hi = min(B, c_lo + chunk);

  if (tid == 0) ctl->nph = 0;
  stamp_phase(ctl, 100);
  arrive_stamp(d.dbg, 0);
  if (a.phases & 1) {
  // ---- V1: counts, duplicate hash, per-vertex counters ---------------------
  {
    int cnt = 0;
    for (long long i = c_lo + threadIdx.x; i < c_hi; i += blockDim.x) cnt += (a.mods[i].x == kVertIns);
    int tot;
    block_excl_scan(cnt, &tot, s_scan);
    if (threadIdx.x == 0) d.blkcnt[blockIdx.x] = tot;
  }
  if (tid == 0) {
    ctl->err_idx = kNoErr;
    ctl->err_nomem = 0;
    ctl->slab_top0 = ctl->slab_top;
    ctl->ngrow = 0;
    ctl->nreloc = 0;
    ctl->nvdch = 0;
  }
  rr_for(B, [&](long long i) {
    int4 m = a.mods[i];
    const long long lim = n0 + B;
    if ((m.x == kEdgeDel || m.x == kEdgeIns) && m.y >= 0 && m.z >= 0 && m.y < lim && m.z < lim) {
      unsigned long long key = edge_key(m.y, m.z);
      long long s = hslot(key, d.hmask);
      while (true) {
        unsigned long long prev = atomicCAS(d.hkeys + s, ~0ull, key);
        if (prev == ~0ull || prev == key) {
          atomicAdd(d.hcnt + s, 1);
          break;
        }
        s = (s + 1) & d.hmask;
      }
      if (m.x == kEdgeIns && rel_edge(d, m)) {
        if (m.y < d.n_cap) atomicAdd(d.icnt + m.y, 1);
        if (m.z < d.n_cap) atomicAdd(d.icnt + m.z, 1);
      }
    } else if (m.x == kVertDel && m.y >= 0 && m.y < n0) {
      atomicAdd(d.vcnt + m.y, 1);
      d.markD[m.y] = a.epD;
    }
  });
  GRID_SYNC_STAMPED(ctl, 101);

  // ---- V2: validate against the pre-batch state; new IDs; allocate ---------
  long long* s_ins = sm.ins;
  if (warp_id() == 0) {  // one warp sums the per-CTA counts
    long long t = 0, m = 0;
    for (int b = lane_id(); b < (int)gridDim.x; b += 32) {
      int c = __ldcg(d.blkcnt + b);
      t += c;
      if (b < (int)blockIdx.x) m += c;
    }
    t = warp_sum(t);
    m = warp_sum(m);
    if (lane_id() == 0) {
      s_ins[0] = t;
      s_ins[1] = m;
    }
  }
  __syncthreads();
  const long long n_ins = s_ins[0], my_base = s_ins[1];
  if (tid == 0) {
    ctl->n_ins = (int)n_ins;  // read by the host when capacity must grow
    if (n0 + n_ins > d.n_cap) atomicOr(&ctl->err_nomem, 1);  // 1: vertex IDs exhausted
  }
  {  // the j-th VERTEX_INSERT in batch order gets ID n0 + j
    long long base = n0 + my_base;
    for (long long t0 = c_lo; t0 < c_hi; t0 += blockDim.x) {
      long long i = t0 + threadIdx.x;
      int f = (i < c_hi) && a.mods[i].x == kVertIns;
      int tot;
      int ex = block_excl_scan(f, &tot, s_scan);
      if (f) d.newid[i] = (int)(base + ex);
      base += tot;
    }
  }
  const long long nlim = n0 + n_ins;
  rr_for(B, [&](long long i) {
    int4 m = a.mods[i];
    bool ok;
    // Every per-vertex word and the first hash probe the checks may need are
    // loaded up front (independent loads in flight together) instead of
    // behind short-circuit chains: one dependent round trip, then the
    // adjacency search.
    const bool edge = m.x == kEdgeDel || m.x == kEdgeIns;
    const bool yo = (edge || m.x == kVertDel) && m.y >= 0 && m.y < n0;
    const bool zo = edge && m.z >= 0 && m.z < n0;
    bool acty = false, actz = false;
    uint32_t mdy = 0, mdz = 0;
    int dgy = 0, dgz = 0, ldy = 0, ldz = 0, icy = 0, icz = 0;
    long long ofy = 0, ofz = 0;
    if (yo) {
      acty = __ldcg(d.active + m.y);
      mdy = __ldcg(d.markD + m.y);
      const longlong2 r = __ldcg(reinterpret_cast<const longlong2*>(d.vr + m.y));  // one 16-byte record
      ofy = r.x;
      dgy = (int)(unsigned)(unsigned long long)r.y;
      ldy = (int)(r.y >> 32);
    }
    if (zo) {
      actz = __ldcg(d.active + m.z);
      mdz = __ldcg(d.markD + m.z);
      const longlong2 r = __ldcg(reinterpret_cast<const longlong2*>(d.vr + m.z));  // one 16-byte record
      ofz = r.x;
      dgz = (int)(unsigned)(unsigned long long)r.y;
      ldz = (int)(r.y >> 32);
    }
    const bool yr = m.y >= 0 && m.y < d.n_cap, zr = m.z >= 0 && m.z < d.n_cap;
    if (m.x == kEdgeIns) {
      icy = yr ? __ldcg(d.icnt + m.y) : 0;
      icz = zr ? __ldcg(d.icnt + m.z) : 0;
    }
    const int vcy = (m.x == kVertDel && yo) ? __ldcg(d.vcnt + m.y) : 0;
    // first-touch stamps and capacities of an insertion's endpoints (the grow
    // reservations below), in the same round trip as the other words
    uint32_t mgy = a.epG, mgz = a.epG;
    int capy = 0, capz = 0;
    if (m.x == kEdgeIns) {
      if (yr) mgy = __ldcg(d.markG + m.y);
      if (zr) mgz = __ldcg(d.markG + m.z);
      if (yo) capy = __ldcg(d.capv + m.y);
      if (zo) capz = __ldcg(d.capv + m.z);
    }
    unsigned long long hkey = 0, hk0 = 0;
    long long hs = 0;
    int hc0 = 0;
    const long long lim = n0 + B;
    if (edge && m.y >= 0 && m.z >= 0 && m.y < lim && m.z < lim) {
      hkey = edge_key(m.y, m.z);
      hs = hslot(hkey, d.hmask);
      hk0 = __ldcg(d.hkeys + hs);
      hc0 = __ldcg(d.hcnt + hs);
    }
    const bool live_y = yo && acty && mdy != a.epD, live_z = zo && actz && mdz != a.epD;
    auto is_new = [&](int x) { return x >= n0 && x < nlim; };
    auto dup_free = [&]() {  // the edge's hash counter (the key is present: V1 inserted it)
      if (hk0 == hkey) return hc0 == 1;
      long long s = (hs + 1) & d.hmask;
      while (__ldcg(d.hkeys + s) != hkey) s = (s + 1) & d.hmask;
      return __ldcg(d.hcnt + s) == 1;
    };
    auto exists = [&]() {  // search the shorter prefix
      return dgy <= dgz ? thread_find(d.adj, ofy, dgy, m.z) >= 0 : thread_find(d.adj, ofz, dgz, m.y) >= 0;
    };
    const bool rel = !edge || rel_edge(d, m);  // the existence / degree checks belong to the endpoint owners
    if (m.x == kEdgeDel) {
      ok = m.y != m.z && live_y && live_z && dup_free() && (!rel || exists());
    } else if (m.x == kVertDel) {
      ok = yo && acty && vcy == 1;
      if (ok) {  // kVdC-entry work chunks of this deletion
        int nch = max(1, (dgy + kVdC - 1) / kVdC);
        int s = agg_alloc(&ctl->nvdch, nch);
        for (int c = 0; c < nch; c++) d.vdch[s + c] = make_int2(m.y, c);
      }
    } else if (m.x == kVertIns) {
      ok = a.vw_unit ? (m.w == 1) : (m.w >= 1 && m.w <= kVwMax);
    } else if (m.x == kEdgeIns) {
      ok = m.y != m.z && (live_y || is_new(m.y)) && (live_z || is_new(m.z));
      ok = ok && (a.ew_unit ? (m.w == 1) : (m.w >= 1 && m.w <= kEwMax));
      ok = ok && dup_free();
      if (ok && live_y && live_z && rel) ok = !exists();
      if (ok) {
        long long du = (m.y < n0 ? ldy : 0) + icy;
        long long dv = (m.z < n0 ? ldz : 0) + icz;
        ok = (du <= kDegMax || !own(d, m.y)) && (dv <= kDegMax || !own(d, m.z));
      }
    } else {
      ok = false;
    }
    if (!ok) atomicMin((long long*)&ctl->err_idx, i);
    // slots for every endpoint an insertion touches (first touch): both stamp
    // exchanges in flight together, then ONE warp-aggregated reservation
    // round for the grow list, the slab and the relocation list (one
    // dependent atomic trip each instead of three per endpoint)
    bool fy = false, fz = false;
    if (m.x == kEdgeIns && rel) {
      const uint32_t oy = (yr && mgy != a.epG) ? atomicExch(d.markG + m.y, a.epG) : a.epG;
      const uint32_t oz = (zr && mgz != a.epG) ? atomicExch(d.markG + m.z, a.epG) : a.epG;
      fy = oy != a.epG;
      fz = oz != a.epG;  // (m.y == m.z: the second exchange sees the first)
    }
    auto grow_nc = [&](bool f, int x, int dg, int ic, int cap, bool& mv) -> unsigned long long {
      mv = false;
      if (!f) return 0ull;
      const long long need = (x < n0 ? dg : 0) + ic;  // prefix length (incl. tombstones) + insertions
      const long long have = x < n0 ? cap : 0;
      mv = need > have;
      if (!mv) return 0ull;
      const unsigned long long nc = (unsigned long long)(need + max((long long)d.slack_min, need / 4));
      return (nc + 3) & ~3ull;
    };
    bool mvy, mvz;
    const unsigned long long ncy = grow_nc(fy, m.y, dgy, icy, capy, mvy);
    const unsigned long long ncz = grow_nc(fz, m.z, dgz, icz, capz, mvz);
    int bg, br;
    unsigned long long bs;
    agg_alloc3(&ctl->ngrow, (int)fy + (int)fz, (unsigned long long*)&ctl->slab_top, ncy + ncz, &ctl->nreloc,
               (int)mvy + (int)mvz, bg, bs, br);
    auto place = [&](bool f, int x, bool mv, unsigned long long nc) {
      if (!f) return;
      d.glist[bg++] = x;
      long long pk = -1;
      if (mv) {
        const long long no = (long long)bs;
        bs += nc;
        if (no + (long long)nc > d.slot_cap) atomicOr(&ctl->err_nomem, 2);  // 2: adjacency slab exhausted
        pk = (no << 24) | (long long)nc;
        d.rlist[br++] = x;  // M3 / M4 walk only the moving prefixes
      }
      d.reloc[x] = pk;
    };
    place(fy, m.y, mvy, ncy);
    place(fz, m.z, mvz, ncz);
  });
  GRID_SYNC_STAMPED(ctl, 102);
  if (tid == 0 && d.sharded) {  // this rank's verdict, all-reduced (MIN, MAX) before the mutation launch
    ctl->sh_err[0] = ctl->err_idx;
    ctl->sh_err[1] = ctl->err_nomem;
  }
  }  // V1 + V2
  if (!(a.phases & 2)) return true;
  const long long n_ins = ldv(&ctl->n_ins);

  // ---- scratch reset (hash, counters) on both the failure and success paths ---
  long long e_idx = ldv(&ctl->err_idx), e_mem = ldv(&ctl->err_nomem);
  if (d.sharded) {  // the global verdict: every rank rejects or applies the batch alike
    e_idx = ldv(&ctl->sh_err[0]);
    e_mem = ldv(&ctl->sh_err[1]);
  }
  const bool failed = e_idx != kNoErr || e_mem != 0;  // (the host reads sh_err on sharded handles)
  for (long long i = tid; i <= d.hmask; i += nthr) {
    d.hkeys[i] = ~0ull;
    d.hcnt[i] = 0;
  }
  const int ng = ldv(&ctl->ngrow);
  for (long long t = tid; t < ng; t += nthr) d.icnt[d.glist[t]] = 0;
  for (long long i = tid; i < B; i += nthr) {
    int4 m = a.mods[i];
    if (m.x == kVertDel && m.y >= 0 && m.y < n0) d.vcnt[m.y] = 0;
  }
  if (failed) {  // uniform: every CTA read the same error words
    if (tid == 0) {
      ctl->slab_need = ctl->slab_top - ctl->slab_top0;  // what the batch asked for: sizes the compaction
      ctl->slab_top = ctl->slab_top0;
    }
    return false;
  }

  // ---- M12: edge deletions and vertex deletions (tombstones) ---------------
  long long cut_acc = 0, W_acc = 0;
  // edge deletions: one thread per modifier; a search in a prefix longer than
  // 32 entries is done by the whole warp (ballot loop)
  rr_for_warp(B, [&](long long i, bool valid) {
    int4 m = valid ? a.mods[i] : make_int4(-1, 0, 0, 0);
    const bool ed = m.x == kEdgeDel && rel_edge(d, m);
    // search the shorter prefix; the twin gives the reverse slot
    int b0 = m.z;  // the endpoint searched for (in the other's, shorter prefix)
    long long oa = 0;
    int da = 0, du = 0, dv = 0;
    uint8_t pu = 0, pv = 0;
    uint32_t sty = 0, stz = 0;
    if (ed) {  // both records, labels and A stamps in one round trip
      long long ou, ov;
      vr_ldcg(d, m.y, ou, du);
      vr_ldcg(d, m.z, ov, dv);
      pu = ld_part(d.part, m.y);
      pv = ld_part(d.part, m.z);
      sty = __ldcg(d.markA + m.y);
      stz = __ldcg(d.markA + m.z);
      oa = ou;
      if (dv < du) {
        b0 = m.y;
        oa = ov;
      }
      da = min(du, dv);
    }
    long long sa = (ed && da <= 32) ? thread_find(d.adj, oa, da, b0) : -1;
    unsigned hm = __ballot_sync(0xffffffffu, ed && da > 32);
    while (hm) {
      int src = __ffs(hm) - 1;
      hm &= hm - 1;
      long long s = warp_find(d.adj, __shfl_sync(0xffffffffu, oa, src), __shfl_sync(0xffffffffu, da, src),
                              __shfl_sync(0xffffffffu, b0, src));
      if (lane_id() == src) sa = s;
    }
    if (ed) {
      long long sb = __ldcg(d.twin + sa);
      int w = d.adjw ? __ldcg(d.adjw + sa) : 1;
      d.adj[sa] = -1;
      d.adj[sb] = -1;
      atomicSub(&d.vr[m.y].ldeg, 1);
      atomicSub(&d.vr[m.z].ldeg, 1);
      if (pu != kPsi && pv != kPsi && pu != pv && own(d, m.y)) cut_acc -= w;
    }
    if (ed) mark_affected_pair(d, m.y, m.z, a.epA, du, dv, sty, stz);
  });
  // vertex deletions, in kVdC-entry work items (most deleted vertices have
  // degree <= 8: one item each; a hub's items spread over the grid).
  // Few items (<= one per warp of the grid, e.g. C2): one warp per item, a
  // lane per entry -- the shortest dependent chain.  Many items (C4): one
  // thread per item, all of its loads in flight together (measured: C2
  // 0.2047 vs 0.2096 ms, C4 0.780 vs 0.808 ms for the other choice).
  const int nvd = ldv(&ctl->nvdch);
  if (tid == 0 && nvd) path_hit(ctl, nvd <= nwarp ? PA_VDEL_WARP : PA_VDEL_THREAD);
  if (nvd <= nwarp) {
    for (long long t = gwarp; t < nvd; t += nwarp) {
      const int2 ch = __ldcg(d.vdch + t);
      const int u = ch.x;
      long long o;
      int dg;
      vr_ldcg(d, u, o, dg);
      const uint8_t pu = ld_part(d.part, u);
      const int j = ch.y * kVdC + lane_id();
      const int x = (lane_id() < kVdC && j < dg) ? __ldcg(d.adj + o + j) : -1;  // -1: tombstone
      const int w = (x >= 0 && d.adjw) ? __ldcg(d.adjw + o + j) : 1;
      const bool xdel = x >= 0 && __ldcg(d.markD + x) == a.epD;
      const int dx = x >= 0 ? __ldcg(&d.vr[x].deg) : 0;
      const uint32_t stx = x >= 0 ? __ldcg(d.markA + x) : a.epA;  // same round trip as the words above
      const uint8_t px = x >= 0 ? ld_part(d.part, x) : kPsi;
      if (x >= 0 && !xdel) {  // the twin is u's entry in x's prefix
        d.adj[__ldcg(d.twin + o + j)] = -1;
        atomicSub(&d.vr[x].ldeg, 1);
      }
      if (x >= 0) {
        if (pu != kPsi && px != kPsi && pu != px && (!xdel || u < x) && own(d, u)) cut_acc -= w;
      }
      if (x >= 0 && !xdel) mark_affected_pre(d, x, a.epA, dx, stx);
      if (ch.y == 0 && lane_id() == 0) {
        int vwu = d.vw ? __ldcg(d.vw + u) : 1;
        if (pu != kPsi) atomic_add_ll(&ctl->Wp[pu], -(long long)vwu);
        W_acc -= vwu;
      }
    }
  } else rr_for(nvd, [&](long long t) {
    const int2 ch = __ldcg(d.vdch + t);
    const int u = ch.x;
    long long o;
    int dg;
    vr_ldcg(d, u, o, dg);
    const uint8_t pu = ld_part(d.part, u);
    const int j0 = ch.y * kVdC;
    int x[kVdC], w[kVdC], dx[kVdC], tw[kVdC];
    bool xdel[kVdC];
#pragma unroll
    for (int e = 0; e < kVdC; e++) {
      x[e] = j0 + e < dg ? __ldcg(d.adj + o + j0 + e) : -1;  // -1: tombstone from an edge deletion
      w[e] = (x[e] >= 0 && d.adjw) ? __ldcg(d.adjw + o + j0 + e) : 1;
    }
#pragma unroll
    for (int e = 0; e < kVdC; e++) {
      xdel[e] = x[e] >= 0 && __ldcg(d.markD + x[e]) == a.epD;
      dx[e] = x[e] >= 0 ? __ldcg(&d.vr[x[e]].deg) : 0;
      tw[e] = x[e] >= 0 ? __ldcg(d.twin + o + j0 + e) : 0;
    }
#pragma unroll
    for (int e = 0; e < kVdC; e++) {
      if (x[e] < 0) continue;
      uint8_t px = ld_part(d.part, x[e]);
      if (pu != kPsi && px != kPsi && pu != px && (!xdel[e] || u < x[e]) && own(d, u)) cut_acc -= w[e];
      if (!xdel[e]) {  // the twin is u's entry in x's prefix
        d.adj[tw[e]] = -1;
        atomicSub(&d.vr[x[e]].ldeg, 1);
      }
    }
    bool want[kVdC];
#pragma unroll
    for (int e = 0; e < kVdC; e++) want[e] = x[e] >= 0 && !xdel[e];
    mark_affected_chunk<kVdC>(d, x, dx, want, a.epA);
    if (ch.y == 0) {
      int vwu = d.vw ? __ldcg(d.vw + u) : 1;
      if (pu != kPsi) atomic_add_ll(&ctl->Wp[pu], -(long long)vwu);
      W_acc -= vwu;
    }
  });
  GRID_SYNC_STAMPED(ctl, 103);

  // ---- M3: finalize deletions; compact / relocate prefixes; insertions ------
  rr_for(B, [&](long long i) {
    int4 m = a.mods[i];
    if (m.x == kVertDel) {
      d.vr[m.y].deg = 0;
      d.vr[m.y].ldeg = 0;
      d.active[m.y] = 0;
      d.part[m.y] = kDel;
    } else if (m.x == kVertIns) {
      int id = d.newid[i];
      d.active[id] = 1;
      if (d.vw) d.vw[id] = m.w;
      d.part[id] = kPsi;  // Alg. 3 L2-5: straight to the pseudo-partition
      d.oldp[id] = kPsi;  // no part before: its first placement is a label change (delta list)
      if (__ldcg(d.markG + id) != a.epG) {
        d.vr[id].deg = 0;
        d.capv[id] = 0;
        d.vr[id].off = 0;
      }
      d.vr[id].ldeg = 0;
      W_acc += m.w;
      int slot = agg_append(&ctl->npsi[0], true);
      d.psi[0][slot] = id;
    }
  });
  // move a prefix (dropping tombstones) from `src` to the fresh region `dst`;
  // every moved slot's twin is copied and the old slot's twin becomes a
  // forward mark -(new slot + 2), resolved in M4
  auto relocate = [&](int x, long long src, long long dst) {
    const int dg = __ldcg(&d.vr[x].deg);
    int wr = 0;
    for (int b = 0; b < dg; b += 128) {  // 4 loads per lane in flight
      int y[4], w[4], tw[4];
#pragma unroll
      for (int t = 0; t < 4; t++) {
        int j = b + t * 32 + lane_id();
        y[t] = j < dg ? __ldcg(d.adj + src + j) : -1;
        w[t] = (j < dg && d.adjw) ? __ldcg(d.adjw + src + j) : 0;
        tw[t] = y[t] >= 0 ? __ldcg(d.twin + src + j) : 0;
      }
#pragma unroll
      for (int t = 0; t < 4; t++) {
        unsigned keep = __ballot_sync(0xffffffffu, y[t] >= 0);
        if (y[t] >= 0) {
          int pos = wr + __popc(keep & ((1u << lane_id()) - 1u));
          d.adj[dst + pos] = y[t];
          if (d.adjw) d.adjw[dst + pos] = w[t];
          d.twin[dst + pos] = tw[t];
          d.twin[src + b + t * 32 + lane_id()] = -(int)(dst + pos) - 2;
        }
        wr += __popc(keep);
      }
    }
    return wr;
  };
  const int nrl = ldv(&ctl->nreloc);
  if (tid == 0 && nrl) path_hit(ctl, PA_RELOC, nrl);
  for (long long t = gwarp; t < nrl; t += nwarp) {  // growing prefixes move to their new slots
    int x = __ldcg(d.rlist + t);
    long long pk = __ldcg(d.reloc + x);
    long long no = pk >> 24;
    int nc = (int)(pk & 0xffffff);
    int wr = 0;
    if (x < n0) wr = relocate(x, __ldcg(&d.vr[x].off), no);
    if (lane_id() == 0) {
      d.vr[x].off = no;
      d.capv[x] = nc;
      d.vr[x].deg = wr;
      d.icnt[x] = wr;  // moved entries to fix up in M4 (icnt is free again after V2)
    }
  }
  if (tid == 0) {
    ctl->n_total = n0 + n_ins;
    ctl->n_ins = (int)n_ins;
  }
  GRID_SYNC_STAMPED(ctl, 104);

  // ---- M4: edge insertions (Alg. 1): append to the dense prefixes ----------
  rr_for(B, [&](long long i) {
    int4 m = a.mods[i];
    if (m.x != kEdgeIns || !rel_edge(d, m)) return;
    // everything that does not depend on the slot reservations is loaded
    // first (offsets are final after M3; labels; the affected stamps), so
    // the reservations and these loads share one round trip
    const long long oy = __ldcg(&d.vr[m.y].off), oz = __ldcg(&d.vr[m.z].off);
    const uint8_t pu = ld_part(d.part, m.y), pv = ld_part(d.part, m.z);
    const uint32_t sy = __ldcg(d.markA + m.y), sz = __ldcg(d.markA + m.z);
    int pu_pos = atomicAdd(&d.vr[m.y].deg, 1);
    int pv_pos = atomicAdd(&d.vr[m.z].deg, 1);
    atomicAdd(&d.vr[m.y].ldeg, 1);
    atomicAdd(&d.vr[m.z].ldeg, 1);
    long long su = oy + pu_pos, sv = oz + pv_pos;
    d.adj[su] = m.z;
    d.adj[sv] = m.y;
    d.twin[su] = (int)sv;
    d.twin[sv] = (int)su;
    if (d.adjw) {
      d.adjw[su] = m.w;
      d.adjw[sv] = m.w;
    }
    if (pu != kPsi && pv != kPsi && pu != pv && own(d, m.y)) cut_acc += m.w;
    mark_affected_pair(d, m.y, m.z, a.epA, pu_pos + 1, pv_pos + 1, sy, sz);
  });
  // twin fix-ups of moved entries: resolve forward marks of moved partners,
  // then point the partner back at the new slot (idempotent when both moved)
  for (long long t = gwarp; t < nrl; t += nwarp) {
    int x = __ldcg(d.rlist + t);
    const long long o = __ldcg(&d.vr[x].off);
    const int cnt = __ldcg(d.icnt + x);
    for (int j = lane_id(); j < cnt; j += 32) {
      long long s = o + j;
      int tp = __ldcg(d.twin + s);
      int f = __ldcg(d.twin + tp);
      if (f < -1) tp = -f - 2;  // the partner moved too
      d.twin[s] = tp;
      d.twin[tp] = (int)s;
    }
    __syncwarp();
    if (lane_id() == 0) d.icnt[x] = 0;
  }
  block_atomic_add(&ctl->cut, cut_acc, s_red);
  block_atomic_add(&ctl->W, W_acc, s_red);
  stamp_phase(ctl, 199);
  return true;
}

__global__ void __launch_bounds__(kThreads, 2) k_apply(Dev d, ApplyArgs a) {
  cg::grid_group grid = cg::this_grid();
  __shared__ ApplySmem sm;
  apply_body(d, a, grid, sm);
}

}  // namespace igk
