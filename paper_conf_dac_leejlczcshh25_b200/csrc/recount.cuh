// recount.cuh -- S9 cut / part-weight reduction as a TMA-pipelined
// full-store scan (unit edge weights; weighted handles use k_recount).
//
// OPT-IN VARIANT (IGK_RECOUNT=tma at igk_create), kept as the measured
// answer to "stage the tile's records and slab span with bulk async copies":
// on B200 it is 2-4x SLOWER than the direct-gather k_recount (C4 0.98 vs
// 0.25 ms; profiles/r02_s9_recount_ab.txt): the CTA-wide tile hand-off
// (mbarrier waits + __syncthreads) makes every tile wait for its slowest
// vertex, and the staged span carries the slack slots the gathers skip.
//
// The scan is HBM-bound: per tile of kRcT consecutive vertex IDs it needs the
// tile's vertex records, its label window and the slab span holding the
// tile's prefixes.  All three are moved by the bulk-copy engine
// (cp.async.bulk, completion on an mbarrier) into shared memory, several
// tiles ahead of the warps that consume them:
//   iteration j:  records of tile j landed -> span [lo, hi) of its prefixes
//                 -> ONE bulk copy of that span (if it fits kRcAdj slots);
//                 meanwhile the warps count tile j-1 out of shared memory;
//                 then the records of tile j+2 are requested.
// So a CTA keeps records for two tiles and one adjacency span in flight
// without spending registers on them, and the dependent record -> prefix ->
// label chain of the direct gather kernel (k_recount) becomes two
// prefetched hops plus shared-memory reads.  Labels of neighbours inside
// the tile's window [t0 - kRcWin, t0 + kRcT + kRcWin) (the generator's
// sinks sit within +-Geom(256) of their drivers) come from
// shared memory, the others from L1/L2.  A tile whose span is larger than
// kRcAdj slots (hubs, relocated prefixes far apart) is counted with direct
// global gathers, same schedule.  Counting rules = k_recount: edges once
// (x > v), pending vertices own no cut edges, sharded handles count the
// edges whose smaller endpoint they own.
#pragma once
#include "common.cuh"

namespace igk {

constexpr int kRcT = 256;        // vertices per tile = 8 warps x 32 lanes
constexpr int kRcWin = 512;      // label window margin (IDs) on each side of the tile
constexpr int kRcLab = kRcT + 2 * kRcWin;
constexpr int kRcAdj = 4096;     // slab slots one staged span may hold (16 KB)
constexpr int kRcStages = 3;     // record / label stages (tile j+2 requested while j-1 is counted)

struct RcSmem {
  VRec rec[kRcStages][kRcT];
  uint8_t lab[kRcStages][kRcLab];
  int4 adj[2][kRcAdj / 4];
  unsigned long long bar_rec[kRcStages];
  unsigned long long bar_adj[2];
  long long span_lo[2];     // slab slot of adj[b][0]
  int span_ok[2];           // the span of the tile in adj[b] was staged
  long long wlo[kRcStages];  // label window of the stage: IDs [wlo, whi)
  long long whi[kRcStages];
  long long red_lo[kRcT / 32], red_hi[kRcT / 32];
  long long s_wp[256];
  long long s_red[32];
};

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(unsigned long long* bar, int count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive_tx(unsigned long long* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(unsigned long long* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(unsigned long long* bar, uint32_t parity) {
  asm volatile(
      "{\n .reg .pred p;\n WAIT_%=:\n"
      " mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      " @!p bra WAIT_%=;\n}\n" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}
// global -> shared bulk copy (TMA engine), completion counted on `bar`;
// 16-byte aligned addresses, size a multiple of 16
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, unsigned long long* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }

__global__ void __launch_bounds__(kRcT) k_recount_tma(Dev d, long long n, long long* out_cut, long long* out_wp,
                                                      long long* out_cnt) {
  extern __shared__ __align__(128) unsigned char rc_raw[];
  RcSmem& S = *reinterpret_cast<RcSmem*>(rc_raw);
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const long long ntiles = (n + kRcT - 1) / kRcT;
  const long long nloc = (long long)blockIdx.x < ntiles ? (ntiles - blockIdx.x + gridDim.x - 1) / gridDim.x : 0;
  for (int p = tid; p < 256; p += kRcT) S.s_wp[p] = 0;
  if (tid == 0) {
    for (int i = 0; i < kRcStages; i++) mbar_init(&S.bar_rec[i], 1);
    for (int i = 0; i < 2; i++) mbar_init(&S.bar_adj[i], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  const long long lab_cap = d.n_cap & ~15ll;  // the label array holds n_cap bytes
  auto issue_rec = [&](long long j) {         // thread 0: records + label window of local tile j
    const int st = (int)(j % kRcStages);
    const long long t0 = ((long long)blockIdx.x + j * gridDim.x) * kRcT;
    const long long nv = min((long long)kRcT, n - t0);
    const long long wlo = max(0ll, t0 - kRcWin);
    const long long whi = max(wlo, min(t0 + kRcT + kRcWin, lab_cap));
    S.wlo[st] = wlo;
    S.whi[st] = whi;
    fence_proxy_async();  // the stage's earlier generic reads are ordered before the async writes
    mbar_arrive_tx(&S.bar_rec[st], (uint32_t)(nv * 16 + (whi - wlo)));
    bulk_g2s(&S.rec[st][0], d.vr + t0, (uint32_t)(nv * 16), &S.bar_rec[st]);
    if (whi > wlo) bulk_g2s(&S.lab[st][0], d.part + wlo, (uint32_t)(whi - wlo), &S.bar_rec[st]);
  };
  if (tid == 0) {
    if (nloc > 0) issue_rec(0);
    if (nloc > 1) issue_rec(1);
  }
  const bool unit_wp = d.vw == nullptr;
  long long cut = 0, ent = 0, nact = 0;

  // count local tile j (records in stage j % 3, span in adj[j & 1])
  auto count_tile = [&](long long j) {
    const int st = (int)(j % kRcStages), ab = (int)(j & 1);
    const long long t0 = ((long long)blockIdx.x + j * gridDim.x) * kRcT;
    const long long base = t0 + warp * 32;
    const long long v = base + lane;
    const long long wlo = S.wlo[st], whi = S.whi[st];
    auto label = [&](long long x) -> uint8_t {
      return (x >= wlo && x < whi) ? S.lab[st][x - wlo] : __ldg(d.part + x);
    };
    bool act = false;
    uint8_t pv = kPsi;
    int dg = 0, ld = 0;
    long long o = 0;
    if (v < n) {
      pv = label(v);
      act = pv != kDel;
      const VRec r = S.rec[st][v - t0];
      o = r.off;
      dg = r.deg;
      ld = r.ldeg;
    }
    if (!act) {
      pv = kPsi;
      dg = 0;
      ld = 0;
    }
    ent += own(d, v) ? ld : 0;
    nact += act;
    const bool placed = act && pv != kPsi;
    if (unit_wp) {  // equal labels of the warp: one shared atomic per label group
      const unsigned pm = __ballot_sync(0xffffffffu, placed);
      if (placed) {
        const unsigned peers = __match_any_sync(pm, (unsigned)pv);
        if ((peers & ((1u << lane) - 1)) == 0)
          atomicAdd((unsigned long long*)&S.s_wp[pv], (unsigned long long)__popc(peers));
      }
    } else if (placed) {
      acc_add(S.s_wp, pv, vert_w(d.vw, v));
    }
    if (!placed || !own(d, v)) dg = 0;
    const bool staged = S.span_ok[ab];
    if (staged) {
      // the prefix is in shared memory: each thread walks its own vertex
      // (no owner search); a staged span holds <= kRcAdj slots, so the
      // longest walk is bounded
      const int4* p4 = &S.adj[ab][(o - S.span_lo[ab]) >> 2];
      for (int c = 0; 4 * c < dg; c++) {
        const int4 x4 = p4[c];
        const int xs[4] = {x4.x, x4.y, x4.z, x4.w};
#pragma unroll
        for (int i = 0; i < 4; i++) {
          if (4 * c + i < dg && xs[i] > v) {
            const uint8_t q = label(xs[i]);
            cut += q != kPsi && q != pv;
          }
        }
      }
      return;
    }
    // not staged (a hub or far-apart relocated prefixes): k_recount's
    // schedule -- the warp's int4 chunks flattened and dealt lane-strided
    int incl = (dg + 3) >> 2;
#pragma unroll
    for (int sh = 1; sh < 32; sh <<= 1) {
      int t = __shfl_up_sync(0xffffffffu, incl, sh);
      if (lane >= sh) incl += t;
    }
    const int total = __shfl_sync(0xffffffffu, incl, 31);
    const int excl = incl - ((dg + 3) >> 2);
    const long long c0 = o >> 2;
    const int4* g4 = reinterpret_cast<const int4*>(d.adj);
    for (int e0 = 0; e0 < total; e0 += 64) {
      int4 xa[2];
      int vl[2], pl[2], rem[2];
#pragma unroll
      for (int t = 0; t < 2; t++) {
        const int e = e0 + t * 32 + lane;
        int jj = 0;  // owner lane: # lanes with incl <= e
#pragma unroll
        for (int b = 16; b; b >>= 1) {
          int cc = __shfl_sync(0xffffffffu, incl, jj + b - 1);
          if (cc <= e) jj += b;
        }
        const long long oj = __shfl_sync(0xffffffffu, c0, jj);
        const int ej = __shfl_sync(0xffffffffu, excl, jj);
        const int dj = __shfl_sync(0xffffffffu, dg, jj);
        pl[t] = __shfl_sync(0xffffffffu, (int)pv, jj);
        vl[t] = (int)(base + jj);
        const int ci = e - ej;
        rem[t] = e < total ? dj - 4 * ci : 0;
        xa[t] = e < total ? __ldg(g4 + oj + ci) : make_int4(-1, -1, -1, -1);
      }
#pragma unroll
      for (int t = 0; t < 2; t++) {
        const int xs[4] = {xa[t].x, xa[t].y, xa[t].z, xa[t].w};
#pragma unroll
        for (int c = 0; c < 4; c++) {
          if (c < rem[t] && xs[c] > vl[t]) {
            const uint8_t q = label(xs[c]);
            if (q != kPsi && q != (uint8_t)pl[t]) cut += 1;
          }
        }
      }
    }
  };

  for (long long j = 0; j < nloc; j++) {
    const int st = (int)(j % kRcStages), ab = (int)(j & 1);
    mbar_wait(&S.bar_rec[st], (uint32_t)((j / kRcStages) & 1));
    // the span of tile j's prefixes (placed, owned vertices with entries)
    {
      const long long t0 = ((long long)blockIdx.x + j * gridDim.x) * kRcT;
      const long long v = t0 + tid;
      long long lo = 0x7fffffffffffffffll, hi = -1;
      if (v < n) {
        const VRec r = S.rec[st][tid];
        const long long wlo = S.wlo[st];
        const uint8_t p = (v < S.whi[st]) ? S.lab[st][v - wlo] : __ldg(d.part + v);
        if (p != kDel && p != kPsi && r.deg > 0 && own(d, v)) {
          lo = r.off;
          hi = r.off + ((r.deg + 3) & ~3);
        }
      }
#pragma unroll
      for (int o = 16; o; o >>= 1) {
        lo = min(lo, __shfl_xor_sync(0xffffffffu, lo, o));
        hi = max(hi, __shfl_xor_sync(0xffffffffu, hi, o));
      }
      if (lane == 0) {
        S.red_lo[warp] = lo;
        S.red_hi[warp] = hi;
      }
      __syncthreads();
      if (tid == 0) {
        for (int w = 1; w < kRcT / 32; w++) {  // thread 0 holds warp 0's reduction
          lo = min(lo, S.red_lo[w]);
          hi = max(hi, S.red_hi[w]);
        }
        const bool any = hi > lo;
        const bool ok = !any || hi - lo <= kRcAdj;
        S.span_ok[ab] = ok;
        S.span_lo[ab] = any ? lo : 0;
        if (ok && any) {
          fence_proxy_async();
          mbar_arrive_tx(&S.bar_adj[ab], (uint32_t)((hi - lo) * 4));
          bulk_g2s(&S.adj[ab][0], d.adj + lo, (uint32_t)((hi - lo) * 4), &S.bar_adj[ab]);
        } else {
          mbar_arrive(&S.bar_adj[ab]);  // nothing staged: complete the phase
        }
      }
    }
    if (j >= 1) {
      mbar_wait(&S.bar_adj[(j - 1) & 1], (uint32_t)(((j - 1) >> 1) & 1));
      count_tile(j - 1);
    }
    __syncthreads();  // stage (j - 1) % 3 and adj[(j - 1) & 1] are free again
    if (tid == 0 && j + 2 < nloc) issue_rec(j + 2);
  }
  if (nloc > 0) {
    mbar_wait(&S.bar_adj[(nloc - 1) & 1], (uint32_t)(((nloc - 1) >> 1) & 1));
    count_tile(nloc - 1);
  }
  __syncthreads();
  block_atomic_add(out_cut, cut, S.s_red);
  block_atomic_add(out_cnt, ent, S.s_red);
  block_atomic_add(out_cnt + 1, nact, S.s_red);
  for (int p = tid; p < d.k; p += kRcT)
    if (S.s_wp[p]) atomicAdd((unsigned long long*)&out_wp[p], (unsigned long long)S.s_wp[p]);
}

}  // namespace igk
