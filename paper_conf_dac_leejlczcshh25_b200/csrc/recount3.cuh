// recount3.cuh -- S9 cut / part-weight reduction: the default
// full-store scan since round 2 (k_recount3; the round-1 kernel k_recount and
// the TMA variant stay selectable for A/B: IGK_RECOUNT=gather / tma).
//
// What bounded the round-1 gather kernel (ncu, C4, profiles/r02_q_*): 124 M
// warp instructions for 10 M vertices (~400 per 32-vertex tile: the per-chunk
// owner search, 10 shuffles per chunk slot), 56% issue slots busy, and 22% of
// the elapsed cycles with idle SMs at the end (statically strided tiles; a
// tile holding a hub of 6,747 neighbours kept one warp busy for ~27 dependent
// trips).  This kernel removes both:
//
//  * Dynamic tiles: a warp takes the next tile of kR3T = 128 consecutive IDs
//    from a global counter (one atomic per 128 vertices).  Lane l holds the
//    vertices base + 32 j + l (j < 4): four coalesced 16-byte record loads.
//  * In-thread prefixes: a vertex's first 4 entries (one int4 chunk -- 75%
//    of the vertices of the circuit graphs have degree <= 4)
//    are read and counted by its own lane with no shuffles at all (two
//    chunks in-thread measured slower: 0.140 vs 0.130 ms at C4).
//  * Residual: the entries beyond 4 of vertices with degree <= kR3Big are
//    listed in shared memory (warp-private) with an inclusive chunk prefix;
//    the warp deals them lane-strided, owner found by a 7-step binary search
//    in shared memory.
//  * Pieces: a vertex with more than kR3Big entries is cut into pieces of
//    kR3Piece entries appended to a global list, counted after a grid barrier
//    by all warps (a piece = 2 dependent trips), so no hub forms a tail.
//
// Counting rules = k_recount: an edge is counted once, by the endpoint with
// the smaller ID (x > v); pending (psi) vertices own no cut edges and count
// for no part; sharded handles count the edges whose smaller endpoint they
// own.  Labels are 1-byte gathers that stay in L2 (the label array of C4 is
// 10 MB of the 126 MB L2).
#pragma once
#include "common.cuh"

namespace igk {

#ifndef IGK_R3V
#define IGK_R3V 4
#endif
constexpr int kR3V = IGK_R3V;     // vertices per lane per tile (A/B builds: -DIGK_R3V=...)
constexpr int kR3T = 32 * kR3V;   // vertices per warp tile (consecutive IDs)
#ifndef IGK_R3IN
#define IGK_R3IN 4
#endif
constexpr int kR3In = IGK_R3IN;   // entries counted in-thread per vertex (int4 chunks of 4; A/B: -DIGK_R3IN)
constexpr int kR3InC = kR3In / 4;
constexpr int kR3Big = 256;       // more entries: the vertex is split into global pieces
constexpr int kR3Piece = 1024;    // entries per piece
#ifndef IGK_R3U
#define IGK_R3U 2
#endif
constexpr int kR3U = IGK_R3U;     // residual chunks per lane per trip
constexpr int kR3PU = 4;          // piece chunks per lane per trip
#ifndef IGK_R3MINB
#define IGK_R3MINB 4
#endif
constexpr int kR3Threads = 256;
constexpr int kR3Warps = kR3Threads / 32;

struct R3Smem {
  int4 hv[kR3Warps][kR3T];   // residual vertices: {chunk index of entry 8, vertex, entries beyond 8, label}
  int incl[kR3Warps][kR3T];  // inclusive prefix of their residual chunk counts
  long long s_wp[256];        // weighted handles: per-part vertex weight
  unsigned s_cnt[256];        // unit weights: per-part vertex count (native 32-bit shared atomics)
  long long s_red[32];
};

// counters (zeroed before the launch): [0] next tile, [1] pieces appended, [2] next piece
template <bool kW>
__global__ void __launch_bounds__(kR3Threads, IGK_R3MINB) k_recount3(Dev d, long long n, long long* out_cut, long long* out_wp,
                                                          long long* out_cnt, unsigned long long* ctr,
                                                          int4* pieces) {
  __shared__ R3Smem S;
  cg::grid_group grid = cg::this_grid();
  const int lane = lane_id(), w = warp_id();
  const unsigned lt = (1u << lane) - 1u;
  for (int p = threadIdx.x; p < 256; p += blockDim.x) {
    S.s_wp[p] = 0;
    S.s_cnt[p] = 0;
  }
  __syncthreads();
  const bool unit_wp = d.vw == nullptr;
  const bool sharded = d.nranks > 1;
  const int4* a4 = reinterpret_cast<const int4*>(d.adj);
  const int4* w4 = reinterpret_cast<const int4*>(d.adjw);
  long long cut = 0, ent = 0, nact = 0;
  const unsigned long long ntiles = (unsigned long long)((n + kR3T - 1) / kR3T);

  // the entries of one chunk that vertex v (label pv) owns: x > v and live;
  // cut if the neighbour's label is a part other than pv (pending neighbours
  // count for no part).  No per-entry length mask: every slab slot past a
  // prefix's length is a tombstone (-1 < v) -- the slab is filled with -1 at
  // create and by every compaction, prefixes only grow by appends, and a
  // relocated prefix lands in never-written bump space.
  int cut32 = 0;  // this tile's count (flushed to the 64-bit total per tile)
  auto count_chunk = [&](const int4& xa, const int4& wa, int v, int pv) {
    const int xs[4] = {xa.x, xa.y, xa.z, xa.w};
    uint8_t q[4];
#pragma unroll
    for (int c = 0; c < 4; c++) q[c] = xs[c] > v ? __ldg(d.part + xs[c]) : (uint8_t)pv;
    if (kW) {
      const int ws[4] = {wa.x, wa.y, wa.z, wa.w};
#pragma unroll
      for (int c = 0; c < 4; c++)
        if (q[c] != kPsi && q[c] != (uint8_t)pv) cut32 += ws[c];
    } else {
#pragma unroll
      for (int c = 0; c < 4; c++) cut32 += (q[c] != kPsi && q[c] != (uint8_t)pv) ? 1 : 0;
    }
  };
  const int4 none = make_int4(-1, -1, -1, -1), ones = make_int4(1, 1, 1, 1);

  // (tried and measured slower at C4, profiles/r02_{t,aj}_*: fetching the
  // next tile's index one tile ahead, 0.142 vs 0.139 ms; pairs of adjacent
  // tiles with the second one's records, labels and slab lines prefetched
  // into L2 while the first is counted, 0.137 vs 0.129 ms)
  while (true) {
    unsigned long long t = 0;
    if (lane == 0) t = atomicAdd(ctr, 1ull);
    t = __shfl_sync(0xffffffffu, t, 0);
    if (t >= ntiles) break;
    const long long base = (long long)t * kR3T;
    // ---- trip 1: the tile's vertex records and labels (coalesced)
    longlong2 r[kR3V];
    int pv[kR3V];
#pragma unroll
    for (int j = 0; j < kR3V; j++) {
      const long long v = base + 32 * j + lane;
      if (v < n) {
        pv[j] = __ldg(d.part + v);
        r[j] = __ldg(reinterpret_cast<const longlong2*>(d.vr + v));
      } else {
        pv[j] = kDel;
        r[j] = make_longlong2(0, 0);
      }
    }
    int din[kR3V];  // entries counted in-thread (<= kR3In)
    int nh = 0;     // residual vertices listed (warp-uniform)
#pragma unroll
    for (int j = 0; j < kR3V; j++) {
      const int v = (int)(base + 32 * j + lane);
      const bool act = pv[j] != kDel;  // the label doubles as the active flag
      const bool placed = act && pv[j] != kPsi;
      const bool mine = !sharded || own(d, v);
      const int dg = (int)(unsigned)(unsigned long long)r[j].y;  // prefix length incl. tombstones
      ent += (act && mine) ? (int)(r[j].y >> 32) : 0;               // live degree
      nact += act;
      if (unit_wp) {  // one shared atomic per label group of the warp
        const unsigned pm = __ballot_sync(0xffffffffu, placed);
        if (placed) {
          const unsigned peers = __match_any_sync(pm, (unsigned)pv[j]);
          if ((peers & lt) == 0) atomicAdd(&S.s_cnt[pv[j]], (unsigned)__popc(peers));
        }
      } else if (placed) {
        acc_add(S.s_wp, pv[j], vert_w(d.vw, v));
      }
      const int dgo = (placed && mine) ? dg : 0;  // entries this lane must scan
      const unsigned c0 = (unsigned)((unsigned long long)r[j].x >> 2);
      const bool big = dgo > kR3Big;
      din[j] = big ? 0 : min(dgo, kR3In);
      const int res = big ? 0 : dgo - din[j];
      const unsigned mr = __ballot_sync(0xffffffffu, res > 0);
      if (res > 0) S.hv[w][nh + __popc(mr & lt)] = make_int4((int)(c0 + kR3InC), v, res, pv[j]);
      nh += __popc(mr);
      if (big) {  // rare: pieces of kR3Piece entries for the phase after the grid barrier
        const int np = (dgo + kR3Piece - 1) / kR3Piece;
        const unsigned long long slot = atomicAdd(ctr + 1, (unsigned long long)np);
        for (int i = 0; i < np; i++)
          pieces[slot + i] = make_int4((int)(c0 + i * (kR3Piece / 4)), v, min(kR3Piece, dgo - i * kR3Piece), pv[j]);
      }
      r[j].x = (long long)c0;
    }
    // ---- trip 2: in-thread chunk (entries 0..3 of every vertex)
    int4 xa[kR3V][kR3InC], wa[kR3V][kR3InC];
#pragma unroll
    for (int j = 0; j < kR3V; j++)
#pragma unroll
      for (int c = 0; c < kR3InC; c++) {
        const bool ld = din[j] > 4 * c;
        xa[j][c] = ld ? __ldg(a4 + (unsigned)r[j].x + c) : none;
        wa[j][c] = (kW && ld) ? __ldg(w4 + (unsigned)r[j].x + c) : ones;
      }
    // residual chunk prefix (warp-uniform branch)
    int R = 0;
    if (nh) {
      __syncwarp();
      int cs[kR3V], s = 0;
#pragma unroll
      for (int i = 0; i < kR3V; i++) {
        const int h = kR3V * lane + i;
        cs[i] = h < nh ? (S.hv[w][h].z + 3) >> 2 : 0;
        s += cs[i];
      }
      int inc = s;
#pragma unroll
      for (int sh = 1; sh < 32; sh <<= 1) {
        const int tv = __shfl_up_sync(0xffffffffu, inc, sh);
        if (lane >= sh) inc += tv;
      }
      int run = inc - s;
#pragma unroll
      for (int i = 0; i < kR3V; i++) {
        run += cs[i];
        if (kR3V * lane + i < nh) S.incl[w][kR3V * lane + i] = run;
      }
      R = __shfl_sync(0xffffffffu, inc, 31);
      __syncwarp();
    }
    // residual chunks e0 + 32 u + lane (u < kR3U), owner by binary search
    int4 xr[kR3U], wr[kR3U];
    int vr[kR3U], pr[kR3U];
    auto load_res = [&](int e0) {
#pragma unroll
      for (int u = 0; u < kR3U; u++) {
        const int e = e0 + 32 * u + lane;
        xr[u] = none;
        wr[u] = ones;
        vr[u] = 0;
        pr[u] = kPsi;
        if (e < R) {
          int h = 0;  // owner = #entries with incl <= e (incl strictly increasing)
#pragma unroll
          for (int b = kR3T / 2; b; b >>= 1)
            if (h + b - 1 < nh && S.incl[w][h + b - 1] <= e) h += b;
          const int4 H = S.hv[w][h];
          const int ci = e - (h ? S.incl[w][h - 1] : 0);
          xr[u] = __ldg(a4 + (unsigned)H.x + ci);
          if (kW) wr[u] = __ldg(w4 + (unsigned)H.x + ci);
          vr[u] = H.y;
          pr[u] = H.w;
        }
      }
    };
    // ---- trip 3: labels of the in-thread entries
#pragma unroll
    for (int j = 0; j < kR3V; j++)
#pragma unroll
      for (int c = 0; c < kR3InC; c++) count_chunk(xa[j][c], wa[j][c], (int)(base + 32 * j + lane), pv[j]);
    // ---- residual entries, kR3U chunks per lane per trip
    for (int e0 = 0; e0 < R; e0 += 32 * kR3U) {
      load_res(e0);  // (issuing the first batch before the in-thread gathers measured slower: 133 vs 130 us at C4)
#pragma unroll
      for (int u = 0; u < kR3U; u++) count_chunk(xr[u], wr[u], vr[u], pr[u]);
    }
    cut += cut32;
    cut32 = 0;
    __syncwarp();  // the residual list is rewritten by the next tile
  }

  // ---- pieces of the heavy vertices, after every tile listed its pieces
  grid.sync();
  const unsigned long long npc = __ldcg(ctr + 1);
  while (true) {
    unsigned long long i = 0;
    if (lane == 0) i = atomicAdd(ctr + 2, 1ull);
    i = __shfl_sync(0xffffffffu, i, 0);
    if (i >= npc) break;
    const int4 P = __ldcg(pieces + i);  // written before the barrier by another CTA
    const int nch = (P.z + 3) >> 2;
    for (int e0 = 0; e0 < nch; e0 += 32 * kR3PU) {
      int4 xr[kR3PU], wr[kR3PU];
#pragma unroll
      for (int u = 0; u < kR3PU; u++) {
        const int e = e0 + 32 * u + lane;
        xr[u] = e < nch ? __ldg(a4 + (unsigned)P.x + e) : none;
        wr[u] = (kW && e < nch) ? __ldg(w4 + (unsigned)P.x + e) : ones;
      }
#pragma unroll
      for (int u = 0; u < kR3PU; u++) count_chunk(xr[u], wr[u], P.y, P.w);
    }
    cut += cut32;
    cut32 = 0;
  }
  block_atomic_add(out_cut, cut, S.s_red);
  block_atomic_add(out_cnt, ent, S.s_red);
  block_atomic_add(out_cnt + 1, nact, S.s_red);
  for (int p = threadIdx.x; p < d.k; p += blockDim.x) {
    const long long wp = S.s_wp[p] + (long long)S.s_cnt[p];
    if (wp) atomicAdd((unsigned long long*)&out_wp[p], (unsigned long long)wp);
  }
}

}  // namespace igk
