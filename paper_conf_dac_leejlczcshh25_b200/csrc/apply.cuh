// apply.cuh -- S1: validate and apply one modifier batch on the device.
//
// One persistent cooperative kernel; phases are separated by grid barriers:
//   V0 clear scratch | V1 dup hash, counts | V2 validate, new IDs, allocate
//   M0 relocate      | M1 edge deletions   | M2 vertex deletions
//   M3 finalize deletions, compact, vertex insertions | M4 edge insertions
// Semantics: reading S1 of P:94-98, Alg. 1-2 and Alg. 3 L1-7.
// Differences from the paper's design: dense-prefix adjacency
// with slack instead of 32-slot buckets; one directed update per thread or
// warp after a validation pass, so concurrent updates of one vertex are
// race-free (the paper's warp-per-modifier bucket insert races, Q10).
#pragma once
#include "common.cuh"

namespace igk {

struct ApplyArgs {
  const int4* mods;
  long long B;
  long long n0;         // n_total before the batch
  uint32_t epD, epT, epG, epA;
  int vw_unit, ew_unit;
};

__device__ __forceinline__ unsigned long long edge_key(int u, int v) {
  unsigned a = (unsigned)min(u, v), b = (unsigned)max(u, v);
  return ((unsigned long long)a << 32) | b;
}
__device__ __forceinline__ long long hslot(unsigned long long key, long long mask) {
  unsigned long long h = key * 0x9E3779B97F4A7C15ull;
  return (long long)(h >> 17) & mask;
}

// linear search of x in the dense prefix of u (thread-sequential)
__device__ __forceinline__ bool has_edge_seq(const Dev& d, int u, int x) {
  long long o = __ldcg(d.off + u);
  int dg = __ldcg(d.deg + u);
  for (int i = 0; i < dg; i++)
    if (__ldcg(d.adj + o + i) == x) return true;
  return false;
}

// warp-cooperative search of x in u's prefix; returns slot index or -1
__device__ __forceinline__ long long warp_find(const Dev& d, int u, int x) {
  long long o = __ldcg(d.off + u);
  int dg = __ldcg(d.deg + u);
  for (int b = 0; b < dg; b += 32) {
    int i = b + lane_id();
    bool hit = i < dg && __ldcg(d.adj + o + i) == x;
    unsigned m = __ballot_sync(0xffffffffu, hit);
    if (m) return o + b + __ffs(m) - 1;
  }
  return -1;
}

__device__ __forceinline__ void mark_affected(const Dev& d, int x, uint32_t epA) {
  bool add = stamp_insert(d.markA, x, epA);
  int slot = agg_append(&d.ctl->nA, add);
  if (add) d.Alist[slot] = x;
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

__global__ void __launch_bounds__(kThreads) k_apply(Dev d, ApplyArgs a) {
  cg::grid_group grid = cg::this_grid();
  __shared__ int s_scan[64];
  __shared__ long long s_red[32];
  Ctl* ctl = d.ctl;
  const long long tid = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  const long long nthr = (long long)gridDim.x * blockDim.x;
  const long long gwarp = tid >> 5, nwarp = nthr >> 5;
  const long long B = a.B, n0 = a.n0;
  const long long chunk = (B + gridDim.x - 1) / gridDim.x;
  const long long c_lo = min(B, (long long)blockIdx.x * chunk), c_hi = min(B, c_lo + chunk);

  // ---- V0: clear the duplicate hash; reset the error word -------------------
  for (long long i = tid; i <= d.hmask; i += nthr) {
    d.hkeys[i] = ~0ull;
    d.hcnt[i] = 0;
  }
  if (tid == 0) {
    ctl->err_idx = kNoErr;
    ctl->err_nomem = 0;
    ctl->slab_top0 = ctl->slab_top;
    ctl->ngrow = 0;
    ctl->ndirty = 0;
  }
  grid.sync();

  // ---- V1: count VERTEX_INSERTs per block chunk, hash edge keys, count ------
  {
    int cnt = 0;
    for (long long i = c_lo + threadIdx.x; i < c_hi; i += blockDim.x) cnt += (a.mods[i].x == kVertIns);
    int tot;
    block_excl_scan(cnt, &tot, s_scan);
    if (threadIdx.x == 0) d.blkcnt[blockIdx.x] = tot;
  }
  for (long long i = tid; i < B; i += nthr) {
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
      if (m.x == kEdgeIns) {
        if (m.y < d.n_cap) atomicAdd(d.icnt + m.y, 1);
        if (m.z < d.n_cap) atomicAdd(d.icnt + m.z, 1);
      }
    } else if (m.x == kVertDel && m.y >= 0 && m.y < n0) {
      atomicAdd(d.vcnt + m.y, 1);
      d.markD[m.y] = a.epD;
    }
  }
  grid.sync();

  // ---- V2: validate against the pre-batch state; new IDs; allocate slots ----
  long long n_ins = 0, my_base = 0;
  for (int b = 0; b < (int)gridDim.x; b++) {
    int c = __ldcg(d.blkcnt + b);
    n_ins += c;
    if (b < (int)blockIdx.x) my_base += c;
  }
  if (tid == 0 && n0 + n_ins > d.n_cap) ctl->err_nomem = 1;
  {  // IDs of VERTEX_INSERTs: the j-th insertion in batch order gets n0 + j
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
  for (long long i = tid; i < B; i += nthr) {
    int4 m = a.mods[i];
    bool ok;
    auto old_live = [&](int x) {
      return x >= 0 && x < n0 && __ldcg(d.active + x) && __ldcg(d.markD + x) != a.epD;
    };
    auto is_new = [&](int x) { return x >= n0 && x < nlim; };
    auto dup_free = [&](int u, int v) {
      unsigned long long key = edge_key(u, v);
      long long s = hslot(key, d.hmask);
      while (d.hkeys[s] != key) s = (s + 1) & d.hmask;
      return __ldcg(d.hcnt + s) == 1;
    };
    auto exists = [&](int u, int v) {  // scan the shorter list
      return __ldcg(d.deg + u) <= __ldcg(d.deg + v) ? has_edge_seq(d, u, v) : has_edge_seq(d, v, u);
    };
    if (m.x == kEdgeDel) {
      ok = m.y != m.z && old_live(m.y) && old_live(m.z) && dup_free(m.y, m.z) && exists(m.y, m.z);
    } else if (m.x == kVertDel) {
      ok = m.y >= 0 && m.y < n0 && __ldcg(d.active + m.y) && __ldcg(d.vcnt + m.y) == 1;
    } else if (m.x == kVertIns) {
      ok = a.vw_unit ? (m.w == 1) : (m.w >= 1 && m.w <= kVwMax);
    } else if (m.x == kEdgeIns) {
      bool uo = old_live(m.y), vo = old_live(m.z);
      ok = m.y != m.z && (uo || is_new(m.y)) && (vo || is_new(m.z));
      ok = ok && (a.ew_unit ? (m.w == 1) : (m.w >= 1 && m.w <= kEwMax));
      ok = ok && dup_free(m.y, m.z);
      if (ok && uo && vo) ok = !exists(m.y, m.z);
      if (ok) {
        long long du = (m.y < n0 ? __ldcg(d.deg + m.y) : 0) + __ldcg(d.icnt + m.y);
        long long dv = (m.z < n0 ? __ldcg(d.deg + m.z) : 0) + __ldcg(d.icnt + m.z);
        ok = du <= kDegMax && dv <= kDegMax;
      }
    } else {
      ok = false;
    }
    if (!ok) atomicMin((long long*)&ctl->err_idx, i);
    // slot allocation for every endpoint an insertion touches (first touch)
    if (m.x == kEdgeIns) {
      int ends[2] = {m.y, m.z};
      for (int e = 0; e < 2; e++) {
        int x = ends[e];
        if (x < 0 || x >= d.n_cap) continue;
        bool first = stamp_insert(d.markG, x, a.epG);
        int slot = agg_append(&ctl->ngrow, first);
        if (!first) continue;
        d.glist[slot] = x;
        long long need = (x < n0 ? __ldcg(d.deg + x) : 0) + __ldcg(d.icnt + x);
        long long have = x < n0 ? __ldcg(d.capv + x) : 0;
        long long pk = -1;
        if (need > have) {
          long long nc = need + max((long long)d.slack_min, need / 4);
          nc = (nc + 3) & ~3ll;
          long long no = atomicAdd((unsigned long long*)&ctl->slab_top, (unsigned long long)nc);
          if (no + nc > d.slot_cap) ctl->err_nomem = 1;
          pk = (no << 24) | nc;
        }
        d.reloc[x] = pk;
      }
    }
  }
  grid.sync();

  const bool failed = ldv(&ctl->err_idx) != kNoErr || ldv(&ctl->err_nomem) != 0;
  // ---- M0: relocate overflowing prefixes (or roll back on failure) ----------
  {
    const int ng = ldv(&ctl->ngrow);
    for (long long t = gwarp; t < ng; t += nwarp) {
      int x = d.glist[t];
      long long pk = d.reloc[x];
      if (lane_id() == 0) d.icnt[x] = 0;
      if (failed || pk < 0) continue;
      long long no = pk >> 24;
      int nc = (int)(pk & 0xffffff);
      if (x < n0) {
        long long o = __ldcg(d.off + x);
        int dg = __ldcg(d.deg + x);
        for (int i = lane_id(); i < dg; i += 32) {
          d.adj[no + i] = __ldcg(d.adj + o + i);
          if (d.adjw) d.adjw[no + i] = __ldcg(d.adjw + o + i);
        }
      } else if (lane_id() == 0) {
        d.deg[x] = 0;
      }
      if (lane_id() == 0) {
        d.off[x] = no;
        d.capv[x] = nc;
      }
    }
    for (long long i = tid; i < B; i += nthr) {
      int4 m = a.mods[i];
      if (m.x == kVertDel && m.y >= 0 && m.y < n0) d.vcnt[m.y] = 0;
    }
    if (failed) {  // uniform: every block saw the same error words
      if (tid == 0) ctl->slab_top = ctl->slab_top0;  // give back the allocations
      return;
    }
  }
  grid.sync();

  long long cut_acc = 0;
  // ---- M1: edge deletions ------------------------------------------
  for (long long i = gwarp; i < B; i += nwarp) {
    int4 m = a.mods[i];
    if (m.x != kEdgeDel) continue;
    long long su = warp_find(d, m.y, m.z);
    long long sv = warp_find(d, m.z, m.y);
    if (lane_id() == 0) {
      int w = d.adjw ? __ldcg(d.adjw + su) : 1;
      d.adj[su] = -1;
      d.adj[sv] = -1;
      uint8_t pu = ld_part(d.part, m.y), pv = ld_part(d.part, m.z);
      if (pu != kPsi && pv != kPsi && pu != pv) cut_acc -= w;
    }
    int ends[2] = {m.y, m.z};
    for (int e = 0; e < 2; e++) {
      if (lane_id() == 0) {
        int x = ends[e];
        if (stamp_insert(d.markT, x, a.epT)) d.dlist[atomicAdd(&ctl->ndirty, 1)] = x;
        if (stamp_insert(d.markA, x, a.epA)) d.Alist[atomicAdd(&ctl->nA, 1)] = x;
      }
    }
  }
  grid.sync();

  // ---- M2: vertex deletions (Alg. 2 L4-6, L11-13; both directions, Q12) ----
  long long W_acc = 0;
  for (long long i = gwarp; i < B; i += nwarp) {
    int4 m = a.mods[i];
    if (m.x != kVertDel) continue;
    const int u = m.y;
    const long long o = __ldcg(d.off + u);
    const int dg = __ldcg(d.deg + u);
    const uint8_t pu = ld_part(d.part, u);
    for (int b = 0; b < dg; b += 32) {
      int j = b + lane_id();
      int x = j < dg ? __ldcg(d.adj + o + j) : -1;
      int w = (x >= 0 && d.adjw) ? __ldcg(d.adjw + o + j) : 1;
      unsigned vm = __ballot_sync(0xffffffffu, x >= 0);
      while (vm) {
        int src = __ffs(vm) - 1;
        vm &= vm - 1;
        int xx = __shfl_sync(0xffffffffu, x, src);
        int ww = __shfl_sync(0xffffffffu, w, src);
        bool xdel = __ldcg(d.markD + xx) == a.epD;
        if (!xdel) {
          long long s = warp_find(d, xx, u);
          if (lane_id() == 0) {
            d.adj[s] = -1;
            if (stamp_insert(d.markT, xx, a.epT)) d.dlist[atomicAdd(&ctl->ndirty, 1)] = xx;
            if (stamp_insert(d.markA, xx, a.epA)) d.Alist[atomicAdd(&ctl->nA, 1)] = xx;
          }
        }
        if (lane_id() == 0) {
          uint8_t px = ld_part(d.part, xx);
          if (pu != kPsi && px != kPsi && pu != px && (!xdel || u < xx)) cut_acc -= ww;
        }
      }
    }
    if (lane_id() == 0) {
      int w = d.vw ? __ldcg(d.vw + u) : 1;
      if (pu != kPsi) atomic_add_ll(&ctl->Wp[pu], -(long long)w);
      W_acc -= w;
    }
  }
  grid.sync();

  // ---- M3: finalize deletions; compact dirty prefixes; vertex insertions ----
  for (long long i = tid; i < B; i += nthr) {
    int4 m = a.mods[i];
    if (m.x == kVertDel) {
      d.deg[m.y] = 0;
      d.active[m.y] = 0;
      d.part[m.y] = kDel;
    } else if (m.x == kVertIns) {
      int id = d.newid[i];
      d.active[id] = 1;
      if (d.vw) d.vw[id] = m.w;
      d.part[id] = kPsi;  // Alg. 3 L2-5: straight to the pseudo-partition
      if (__ldcg(d.markG + id) != a.epG) {
        d.deg[id] = 0;
        d.capv[id] = 0;
        d.off[id] = 0;
      }
      W_acc += m.w;
      int slot = atomicAdd(&ctl->npsi[0], 1);
      d.psi[0][slot] = id;
    }
  }
  {
    const int nd = ldv(&ctl->ndirty);
    for (long long t = gwarp; t < nd; t += nwarp) {
      int x = d.dlist[t];
      if (__ldcg(d.markD + x) == a.epD) continue;
      const long long o = __ldcg(d.off + x);
      const int dg = __ldcg(d.deg + x);
      int wr = 0;
      for (int b = 0; b < dg; b += 32) {
        int j = b + lane_id();
        int y = j < dg ? __ldcg(d.adj + o + j) : -1;
        int w = (j < dg && d.adjw) ? __ldcg(d.adjw + o + j) : 0;
        unsigned keep = __ballot_sync(0xffffffffu, y >= 0);
        __syncwarp();
        if (y >= 0) {
          int pos = wr + __popc(keep & ((1u << lane_id()) - 1u));
          d.adj[o + pos] = y;
          if (d.adjw) d.adjw[o + pos] = w;
        }
        wr += __popc(keep);
        __syncwarp();
      }
      if (lane_id() == 0) d.deg[x] = wr;
    }
  }
  if (tid == 0) {
    ctl->n_total = n0 + n_ins;
    ctl->n_ins = (int)n_ins;
  }
  grid.sync();

  // ---- M4: edge insertions (Alg. 1): append to the dense prefix -------------
  for (long long i = tid; i < B; i += nthr) {
    int4 m = a.mods[i];
    if (m.x != kEdgeIns) continue;
    int pu_pos = atomicAdd(d.deg + m.y, 1);
    int pv_pos = atomicAdd(d.deg + m.z, 1);
    long long su = __ldcg(d.off + m.y) + pu_pos, sv = __ldcg(d.off + m.z) + pv_pos;
    d.adj[su] = m.z;
    d.adj[sv] = m.y;
    if (d.adjw) {
      d.adjw[su] = m.w;
      d.adjw[sv] = m.w;
    }
    uint8_t pu = ld_part(d.part, m.y), pv = ld_part(d.part, m.z);
    if (pu != kPsi && pv != kPsi && pu != pv) cut_acc += m.w;
    mark_affected(d, m.y, a.epA);
    mark_affected(d, m.z, a.epA);
  }
  block_atomic_add(&ctl->cut, cut_acc, s_red);
  block_atomic_add(&ctl->W, W_acc, s_red);
}

}  // namespace igk
