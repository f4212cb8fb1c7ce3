// igk.cu -- libigk: C ABI (include/igk.h) + create-time / query kernels.
//
// Hot path: k_apply (apply.cuh) and k_refine (refine.cuh), each ONE
// persistent cooperative launch per call.  This file holds the handle, the
// store build (S0), the cut/weight reduction (S9) and the exports.
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <unistd.h>
#include <nccl.h>  // types only: NCCL is loaded at run time (nccl_api), not linked
#include <nvtx3/nvToolsExt.h>

#include <algorithm>
#include <atomic>
#include <cstdio>
#include <cstddef>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <string>
#include <vector>

#include "../../include/igk.h"
#include "apply.cuh"
#include "common.cuh"
#include "fgp.cuh"
#include "recount.cuh"
#include "recount3.cuh"
#include "refine.cuh"
#include "step.cuh"
#include <cub/cub.cuh>
#include <chrono>

using namespace igk;

// igk_step runs batches of at least this many modifiers as two launches
// (k_apply at full occupancy + k_refine) instead of the fused k_step; the
// fused launch wins or ties up to C3-10% batches (~56K modifiers, measured)
constexpr long long kSplitB = 131072;


// ---------------------------------------------------------------------------
// create-time store build: copy every CSR row into its slab prefix
// ---------------------------------------------------------------------------
__global__ void k_build(Dev d, const int64_t* xadj, const int32_t* adjncy, const int32_t* adjwgt, int64_t n) {
  const long long gw = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const long long nw = ((long long)gridDim.x * blockDim.x) >> 5;
  for (long long u = gw; u < n; u += nw) {
    const long long s = xadj[u], e = xadj[u + 1], o = d.vr[u].off;
    for (long long j = s + lane_id(); j < e; j += 32) {
      d.adj[o + j - s] = adjncy[j];
      if (d.adjw) d.adjw[o + j - s] = adjwgt[j];
    }
  }
}

// ---------------------------------------------------------------------------
// S9: cut / part-weight reduction, a full store scan, HBM-bound.
// Work unit = a warp tile of 32 consecutive vertex IDs: the per-vertex arrays
// (active, part, deg, off) are read coalesced, one vertex per lane.  Every
// adjacency prefix starts 16-byte aligned (capacities are multiples of 4), so
// a prefix is a run of int4 chunks; the tile's chunks are flattened (warp
// prefix sum of ceil(deg/4)) and dealt lane-strided, kRcU chunks per lane per
// round trip, so a tile costs ceil(chunks / (32 kRcU)) dependent load trips
// whatever its degree mix -- hubs of 10^4 neighbours and degree-1 leaves share
// one schedule (no divergent per-thread loops).  A chunk's owner lane is found
// by a 5-step shuffle search over the inclusive chunk prefix.  (Measured: a
// variant that first reads every lane's own first chunk without the search
// was slower, C4 282 -> 333 us; so were a search-free path for tiles whose
// prefixes all fit one lane, C4 217 -> 229 us, and a next-tile prefetch of the
// vertex record, no change: profiles/r01_s15_recount_ab.txt.)  Labels are a
// 1-byte gather that stays in L2.  Edges are counted once (x > v); pending
// (psi) vertices own no cut edges and count for no part.
// ---------------------------------------------------------------------------
constexpr int kRcU = 2;  // int4 chunks per lane in flight
__global__ void __launch_bounds__(256) k_recount(Dev d, long long n, long long* out_cut, long long* out_wp,
                                                 long long* out_cnt) {
  __shared__ long long s_wp[256];
  __shared__ long long s_red[32];
  for (int p = threadIdx.x; p < 256; p += blockDim.x) s_wp[p] = 0;
  __syncthreads();
  const int lane = lane_id();
  const bool unit_wp = d.vw == nullptr;  // unit weights: W_p by label-group counts
  long long cut = 0, ent = 0, nact = 0;
  const long long nwarps = ((long long)gridDim.x * blockDim.x) >> 5;
  for (long long base = (((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5) * 32; base < n;
       base += nwarps * 32) {
    const long long v = base + lane;
    bool act = false;
    uint8_t pv = kPsi;
    int dg = 0, ld = 0;
    long long o = 0;
    if (v < n) {
      pv = __ldg(d.part + v);
      act = pv != kDel;  // the label doubles as the active flag
      const longlong2 r = __ldg(reinterpret_cast<const longlong2*>(d.vr + v));  // one 16-byte record
      o = r.x;
      dg = (int)(unsigned)(unsigned long long)r.y;  // prefix length incl. tombstones
      ld = (int)(r.y >> 32);                         // live degree
    }
    if (!act) {
      pv = kPsi;
      dg = 0;
      ld = 0;
    }
    ent += own(d, v) ? ld : 0;  // live adjacency entries (algorithmic bytes of the scan)
    nact += act;
    const bool placed = act && pv != kPsi;
    if (unit_wp) {
      // lanes with the same label form one group; its lowest lane adds the
      // group size (one match + one shared atomic per label present, instead
      // of k ballots per tile: C4 recount 0.275 -> 0.217 ms with the grid below)
      const unsigned pm = __ballot_sync(0xffffffffu, placed);
      if (placed) {
        const unsigned peers = __match_any_sync(pm, (unsigned)pv);
        if ((peers & ((1u << lane) - 1)) == 0)
          atomicAdd((unsigned long long*)&s_wp[pv], (unsigned long long)__popc(peers));
      }
    } else if (placed) {
      acc_add(s_wp, pv, vert_w(d.vw, v));
    }
    if (!placed || !own(d, v)) dg = 0;  // pending vertices own no cut edges; sharded: the owner of the smaller endpoint counts
    // inclusive prefix of the tile's chunk counts
    int incl = (dg + 3) >> 2;
#pragma unroll
    for (int sh = 1; sh < 32; sh <<= 1) {
      int t = __shfl_up_sync(0xffffffffu, incl, sh);
      if (lane >= sh) incl += t;
    }
    const int total = __shfl_sync(0xffffffffu, incl, 31);
    const int excl = incl - ((dg + 3) >> 2);
    const long long c0 = o >> 2;  // chunk index of the prefix start (off is a multiple of 4)
    const int4* a4 = reinterpret_cast<const int4*>(d.adj);
    const int4* w4 = reinterpret_cast<const int4*>(d.adjw);
    for (int e0 = 0; e0 < total; e0 += 32 * kRcU) {
      int4 xa[kRcU], wa[kRcU];
      int vl[kRcU], pl[kRcU], rem[kRcU];
#pragma unroll
      for (int t = 0; t < kRcU; t++) {
        const int e = e0 + t * 32 + lane;
        // owner lane j = #lanes with incl <= e (uniform 5-step search)
        int j = 0;
#pragma unroll
        for (int b = 16; b; b >>= 1) {
          int c = __shfl_sync(0xffffffffu, incl, j + b - 1);
          if (c <= e) j += b;
        }
        const long long oj = __shfl_sync(0xffffffffu, c0, j);
        const int ej = __shfl_sync(0xffffffffu, excl, j);
        const int dj = __shfl_sync(0xffffffffu, dg, j);
        pl[t] = __shfl_sync(0xffffffffu, (int)pv, j);
        vl[t] = (int)(base + j);
        const int ci = e - ej;  // chunk within the owner's prefix
        rem[t] = e < total ? dj - 4 * ci : 0;  // live entries in this chunk (>= 4: all)
        xa[t] = e < total ? __ldg(a4 + oj + ci) : make_int4(-1, -1, -1, -1);
        wa[t] = (e < total && w4) ? __ldg(w4 + oj + ci) : make_int4(1, 1, 1, 1);
      }
      uint8_t q[kRcU][4];
#pragma unroll
      for (int t = 0; t < kRcU; t++) {
        const int xs[4] = {xa[t].x, xa[t].y, xa[t].z, xa[t].w};
#pragma unroll
        for (int c = 0; c < 4; c++) q[t][c] = (c < rem[t] && xs[c] > vl[t]) ? __ldg(d.part + xs[c]) : (uint8_t)pl[t];
      }
#pragma unroll
      for (int t = 0; t < kRcU; t++) {
        const int ws[4] = {wa[t].x, wa[t].y, wa[t].z, wa[t].w};
#pragma unroll
        for (int c = 0; c < 4; c++)
          if (q[t][c] != kPsi && q[t][c] != (uint8_t)pl[t]) cut += ws[c];
      }
    }
  }
  block_atomic_add(out_cut, cut, s_red);
  block_atomic_add(out_cnt, ent, s_red);
  block_atomic_add(out_cnt + 1, nact, s_red);
  for (int p = threadIdx.x; p < d.k; p += blockDim.x)
    if (s_wp[p]) atomicAdd((unsigned long long*)&out_wp[p], (unsigned long long)s_wp[p]);
}

// ---------------------------------------------------------------------------
// store maintenance: compaction of the slab into fresh arrays.
// Relocations leave holes and tombstones stay until a prefix moves; this
// copies every live entry to a new dense layout (warp per vertex), recording
// old slot -> new slot, then rewrites every twin through that map.
// ---------------------------------------------------------------------------
__global__ void k_compact_copy(Dev d, long long n, const int64_t* noff, int32_t* nadj, int32_t* nadjw,
                               int32_t* ntwin, int32_t* fwd) {
  const long long gw = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const long long nw = ((long long)gridDim.x * blockDim.x) >> 5;
  for (long long v = gw; v < n; v += nw) {
    const long long o = d.vr[v].off, no = noff[v];
    const int dg = d.active[v] ? d.vr[v].deg : 0;
    int wr = 0;
    for (int b = 0; b < dg; b += 32) {
      int j = b + lane_id();
      int y = j < dg ? d.adj[o + j] : -1;
      unsigned keep = __ballot_sync(0xffffffffu, y >= 0);
      if (y >= 0) {
        long long pos = no + wr + __popc(keep & ((1u << lane_id()) - 1u));
        nadj[pos] = y;
        if (nadjw) nadjw[pos] = d.adjw[o + j];
        ntwin[pos] = d.twin[o + j];  // still an old slot: rewritten below
        fwd[o + j] = (int32_t)pos;
      }
      wr += __popc(keep);
    }
  }
}
__global__ void k_compact_twins(long long used, const int32_t* nadj, int32_t* ntwin, const int32_t* fwd) {
  for (long long s = (long long)blockIdx.x * blockDim.x + threadIdx.x; s < used;
       s += (long long)gridDim.x * blockDim.x)
    if (nadj[s] >= 0) ntwin[s] = fwd[ntwin[s]];
}

// igk_num_vertices: active vertices (the label doubles as the active flag)
__global__ void k_count_active(Dev d, long long n, long long* out) {
  long long c = 0;
  for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (long long)gridDim.x * blockDim.x)
    c += d.part[v] != kDel;
  c = warp_sum(c);
  if (lane_id() == 0 && c) atomicAdd((unsigned long long*)out, (unsigned long long)c);
}
// igk_export_csr: live degree of every ID (deleted rows are empty, I6)
__global__ void k_export_deg(Dev d, long long n, long long* ldeg) {
  for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (long long)gridDim.x * blockDim.x)
    ldeg[v] = d.part[v] != kDel ? d.vr[v].ldeg : 0;
}
// igk_export_csr: the live entries of every prefix (tombstones dropped, slot
// order kept) gathered into one dense CSR on the device -- one warp per row
__global__ void k_export_rows(Dev d, long long n, const long long* xoff, int32_t* oadj, int32_t* ow) {
  const long long gw = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const long long nw = ((long long)gridDim.x * blockDim.x) >> 5;
  for (long long v = gw; v < n; v += nw) {
    if (d.part[v] == kDel) continue;
    const long long o = d.vr[v].off, base = xoff[v];
    const int dg = d.vr[v].deg;
    int wr = 0;
    for (int b = 0; b < dg; b += 32) {
      const int j = b + lane_id();
      const int y = j < dg ? d.adj[o + j] : -1;
      const unsigned keep = __ballot_sync(0xffffffffu, y >= 0);
      if (y >= 0) {
        const long long pos = base + wr + __popc(keep & ((1u << lane_id()) - 1u));
        oadj[pos] = y;
        ow[pos] = d.adjw ? d.adjw[o + j] : 1;
      }
      wr += __popc(keep);
    }
  }
}

// igk_repartition: the active vertices relabelled densely in ID order (act =
// 0/1 flags, did = their exclusive prefix sum), live rows gathered with
// dense neighbour IDs (then row-sorted), the FGP partition installed back
__global__ void k_rp_flag(Dev d, long long n, int32_t* act, int* npsi) {
  int c = 0;
  for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (long long)gridDim.x * blockDim.x) {
    const bool a = d.active[v] != 0;
    act[v] = a;
    c += a && d.part[v] == kPsi;
  }
  if (c) atomicAdd(npsi, c);
}
__global__ void k_rp_deg(Dev d, long long n, const int32_t* act, const int32_t* did, long long* cdeg, int32_t* cvw) {
  for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (long long)gridDim.x * blockDim.x)
    if (act[v]) {
      cdeg[did[v]] = d.vr[v].ldeg;
      cvw[did[v]] = d.vw ? d.vw[v] : 1;
    }
}
__global__ void k_rp_rows(Dev d, long long n, const int32_t* act, const int32_t* did, const long long* cx,
                          int32_t* cadj, int32_t* cw) {
  const long long gw = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const long long nw = ((long long)gridDim.x * blockDim.x) >> 5;
  for (long long v = gw; v < n; v += nw) {
    if (!act[v]) continue;
    const long long o = d.vr[v].off, base = cx[did[v]];
    const int dg = d.vr[v].deg;
    int wr = 0;
    for (int b = 0; b < dg; b += 32) {
      const int j = b + lane_id();
      const int y = j < dg ? d.adj[o + j] : -1;
      const unsigned keep = __ballot_sync(0xffffffffu, y >= 0);
      if (y >= 0) {
        const long long pos = base + wr + __popc(keep & ((1u << lane_id()) - 1u));
        cadj[pos] = did[y];
        cw[pos] = d.adjw ? d.adjw[o + j] : 1;
      }
      wr += __popc(keep);
    }
  }
}
__global__ void k_rp_install(Dev d, long long n, const int32_t* act, const int32_t* did, const int32_t* dpart) {
  for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (long long)gridDim.x * blockDim.x)
    if (act[v]) d.part[v] = (uint8_t)dpart[did[v]];
}

__global__ void k_export_part(Dev d, long long n, int32_t* out) {
  for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (long long)gridDim.x * blockDim.x) {
    uint8_t p = d.part[v];
    out[v] = !d.active[v] ? -1 : (p == kPsi ? -2 : (int)p);
  }
}

// ---------------------------------------------------------------------------
// handle
// ---------------------------------------------------------------------------
struct igk_graph {
  int device = 0;
  int recount_blocks = 0;    // k_recount grid (occupancy-derived at create)
  int recount_tma_blocks = 0;  // k_recount_tma grid (unit edge weights)
  int recount_tma = 0;       // S9 kernel: k_recount3 (0), the round-1 gathers (2; IGK_RECOUNT=gather) or the TMA variant (1; IGK_RECOUNT=tma)
  int recount3_blocks = 0;   // k_recount3 grid (cooperative: co-resident CTAs), unit edge weights
  int recount3w_blocks = 0;  // the same, weighted handles
  long long n_grow = 0;      // vertex-array growths (host path counter)
  long long n_split = 0;     // igk_step launches as k_apply + k_refine (batch >= split_b)
  long long n_fused = 0;     // igk_step launches as one k_step
  long long n_notice_fallback = 0;  // fast-path steps that fell back to the copy + sync
  // sharding (igk_options.nranks > 1)
  bool wide = false;           // wide-weight handle (NEXT-2 coarse levels): refine only, no modifiers
  bool refine_due = false;     // a batch was applied and not yet refined (igk_repartition refuses)
  long long fallback_ppm = 0;  // igk_options.fgp_fallback_ppm (0 = off)
  long long mods_since_full = 0, n_at_full = 0;  // the fallback policy's counters
  bool delta_replaced = false; // igk_repartition replaced the partition: no delta until the next refine
  int nranks = 1, rank = 0;
  bool sharded = false;        // the sharded protocol (nranks > 1, or a transport given for one rank)
  igk_comm comm{};             // host-callback transport (when no NCCL communicator)
  void* nccl = nullptr;        // ncclComm_t created from igk_options.nccl_id
  void* xp_host = nullptr;     // pinned staging of the callback transport
  size_t xp_host_cap = 0;
  long long* d_xp = nullptr;   // kXpWords-word device scratch for host-value all-reduces
  long long cut_total = 0;     // sharded: the global cut (sum of the ranks' partial cuts)
  void* sort_tmp = nullptr;    // sharded: CUB radix-sort scratch (canonical pending list)
  size_t sort_tmp_cap = 0;
  // NEXT-3 persistent P2P rounds (igk_options.p2p)
  bool p2p = false;
  int ranks_per_device = 1;
  int grid_p2p = 0;
  int4* p2p_mem = nullptr;                 // this rank's two record buffers (2 x n_cap int4)
  unsigned long long* p2p_bar = nullptr;   // this rank's barrier counter
  long long p2p_cap = 0;                   // entries per buffer
  int4* p2p_bufs[8][2] = {};               // every rank's buffers (own, peer or IPC-mapped)
  unsigned long long* p2p_bars[8] = {};
  bool p2p_ipc[8] = {};                    // mapped with cudaIpcOpenMemHandle (closed on teardown)
  long long p2p_rounds = 0;                // rounds run so far (barrier counter base / n)
  cudaStream_t stream = nullptr;
  bool poisoned = false;
  std::string err;
  Dev d{};
  long long e_ppm = 0;
  int vw_unit = 1, ew_unit = 1;
  uint32_t epoch = 1;   // last stamp value handed out
  uint32_t epochA = 0;  // stamp of the current affected set
  int grid_apply = 0, grid_refine = 0;
  int grid_refine_k = 0;     // k_refine alone (igk_refine, split step): its own occupancy
  int grid_apply_wide = 0;   // k_apply at full occupancy (split step of large batches)
  long long split_b = 0;     // igk_step: batches of >= split_b modifiers run k_apply + k_refine
  size_t smem_refine = 0, smem_step = 0;
  long long launches = 0;
  igk_modifier* h_stage = nullptr;  // pinned staging for host batches
  long long h_stage_cap = 0;
  int4* d_mods = nullptr;
  long long d_mods_cap = 0;
  long long newid_cap = 0;
  int check = 0;
  int debug_phases = 0;
  int prof = 0;  // profile mode (igk_debug_set_profile): phase stamps + per-phase work counters
  long long compactions = 0;
  // pipelined steps (igk_stage_batch / igk_step_begin / igk_step_end): two
  // device batch buffers filled on a copy stream while a step runs
  cudaStream_t copy_stream = nullptr;
  int4* sd_mods[2] = {nullptr, nullptr};
  long long sd_cap[2] = {0, 0}, sd_count[2] = {0, 0};
  igk_modifier* sh_stage[2] = {nullptr, nullptr};
  long long sh_cap[2] = {0, 0};
  cudaEvent_t ev_stage[2] = {};
  int staged = -1, stage_next = 0, inflight = 0, inflight_buf = 0;
  bool inflight_posted = false;
  long long inflight_n0 = 0;
  long long hash_cap = 0;
  int32_t* d_out = nullptr;  // export buffer
  long long* d_red = nullptr;  // recount outputs: [0] cut, [1..256] Wp, [257] entries, [258] active, [259..261] k_recount3 counters
  long long last_entries = 0, last_active = 0;
  Ctl* h_ctl = nullptr;        // pinned mirror of the control block
  Ctl* h_map = nullptr;        // host-mapped output head written by the kernel (igk_step fast path)
  unsigned* h_flag = nullptr;  // host-mapped completion notice
  unsigned seq = 0;            // last notice value
  int ms_pending = 0;          // ev[0] -> ev[1] not yet converted (fast path returns before ev[1])
  cudaEvent_t ev[6] = {};
  float ms_refine = 0, ms_apply = 0, ms_recount = 0;
  std::vector<void*> allocs;
  std::vector<std::pair<int, unsigned long long>> ph[2];  // phase stamps: [0] apply, [1] refine
};

namespace {

thread_local std::string t_create_err;  // why the last igk_create of this thread failed (igk_last_error(NULL))

// Every entry point runs on the handle's device and restores the caller's
// current device on return (the ABI allows handles on several GPUs).
struct DevGuard {
  int prev = -1;
  explicit DevGuard(int dev) {
    int cur = -1;
    if (cudaGetDevice(&cur) == cudaSuccess && cur != dev && cudaSetDevice(dev) == cudaSuccess) prev = cur;
  }
  ~DevGuard() {
    if (prev >= 0) cudaSetDevice(prev);
  }
};
// NVTX range around each entry point (visible in nsys / ncu timelines)
struct NvtxRange {
  explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
  ~NvtxRange() { nvtxRangePop(); }
};
#define ENTRY(g, name)             \
  DevGuard igk_dg_((g)->device);   \
  NvtxRange igk_nv_(name)

igk_status fail(igk_graph* g, igk_status s, const std::string& msg) {
  if (g) g->err = msg;
  return s;
}

bool cuda_ok(igk_graph* g, cudaError_t e, const char* what) {
  if (e == cudaSuccess) return true;
  if (g) {
    g->poisoned = true;
    g->err = std::string(what) + ": " + cudaGetErrorString(e);
  }
  return false;
}

#define CK(call)                                            \
  do {                                                      \
    if (!cuda_ok(g, (call), #call)) return IGK_ECUDA;       \
  } while (0)

template <class T>
bool dalloc(igk_graph* g, T** p, size_t count) {
  void* q = nullptr;
  if (cudaMalloc(&q, std::max<size_t>(count, 1) * sizeof(T)) != cudaSuccess) return false;
  g->allocs.push_back(q);
  *p = (T*)q;
  return true;
}

uint32_t next_epoch(igk_graph* g) { return ++g->epoch; }

// capacities grow geometrically so that slowly growing batches do not
// re-allocate (pinned host allocations are expensive)
long long grow_cap(long long need) {
  long long c = 1024;
  while (c < need) c <<= 1;
  return c;
}

// strided copies between the packed per-vertex records and a plain array of
// one field (host or device side)
static cudaError_t vr_put(VRec* vr, size_t field, const void* src, size_t elem, long long n, cudaMemcpyKind kind,
                          cudaStream_t s) {
  if (n <= 0) return cudaSuccess;
  return cudaMemcpy2DAsync((char*)vr + field, sizeof(VRec), src, elem, elem, (size_t)n, kind, s);
}
static cudaError_t vr_get(void* dst, const VRec* vr, size_t field, size_t elem, long long n, cudaMemcpyKind kind,
                          cudaStream_t s) {
  if (n <= 0) return cudaSuccess;
  return cudaMemcpy2DAsync(dst, elem, (const char*)vr + field, sizeof(VRec), elem, (size_t)n, kind, s);
}

int coop_grid(const void* fn, size_t smem, int want_per_sm, int dev) {
  int sms = 0, occ = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, fn, kThreads, smem);
  if (occ < 1) occ = 1;
  int per = want_per_sm > 0 ? std::min(want_per_sm, occ) : 1;
  return sms * per;
}

// ---------------------------------------------------------------------------
// collectives of sharded handles: NCCL (loaded at run time) or the host
// callback of igk_options.comm.  Every all-reduce is in place on DEVICE
// memory, ordered on the handle's stream.
// ---------------------------------------------------------------------------
struct NcclApi {
  decltype(&ncclGetUniqueId) get_unique_id = nullptr;
  decltype(&ncclCommInitRank) init_rank = nullptr;
  decltype(&ncclAllReduce) all_reduce = nullptr;
  decltype(&ncclCommDestroy) destroy = nullptr;
  decltype(&ncclGetErrorString) error_string = nullptr;
};
const NcclApi* nccl_api() {
  static NcclApi api;
  static bool ok = false;
  static std::once_flag once;
  std::call_once(once, [] {
    void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);  // the copy torch already loaded, if any
    if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
    if (!h) return;
    api.get_unique_id = (decltype(api.get_unique_id))dlsym(h, "ncclGetUniqueId");
    api.init_rank = (decltype(api.init_rank))dlsym(h, "ncclCommInitRank");
    api.all_reduce = (decltype(api.all_reduce))dlsym(h, "ncclAllReduce");
    api.destroy = (decltype(api.destroy))dlsym(h, "ncclCommDestroy");
    api.error_string = (decltype(api.error_string))dlsym(h, "ncclGetErrorString");
    ok = api.get_unique_id && api.init_rank && api.all_reduce && api.destroy && api.error_string;
  });
  return ok ? &api : nullptr;
}

enum { XP_I64 = 0, XP_U32 = 1 };
constexpr int kXpWords = 512;  // device scratch of host-value all-reduces (p2p blobs: 8 ranks x 40 words)
enum { XP_SUM = 0, XP_MIN = 1, XP_MAX = 2 };
igk_status xp_allreduce(igk_graph* g, void* dptr, long long count, int dtype, int op) {
  if (!g->sharded || count <= 0) return IGK_OK;
  const size_t bytes = (size_t)count * (dtype == XP_I64 ? 8 : 4);
  if (g->nccl) {
    const NcclApi* api = nccl_api();
    const ncclRedOp_t rop = op == XP_SUM ? ncclSum : (op == XP_MIN ? ncclMin : ncclMax);
    ncclResult_t r = api->all_reduce(dptr, dptr, (size_t)count, dtype == XP_I64 ? ncclInt64 : ncclUint32, rop,
                                     (ncclComm_t)g->nccl, g->stream);
    if (r != ncclSuccess) {
      g->poisoned = true;
      return fail(g, IGK_ENCCL, std::string("ncclAllReduce: ") + api->error_string(r));
    }
    return IGK_OK;
  }
  if (bytes > g->xp_host_cap) {
    if (g->xp_host) cudaFreeHost(g->xp_host);
    g->xp_host = nullptr;
    g->xp_host_cap = 0;
    size_t cap = 1 << 16;
    while (cap < bytes) cap <<= 1;
    CK(cudaMallocHost(&g->xp_host, cap));
    g->xp_host_cap = cap;
  }
  CK(cudaMemcpyAsync(g->xp_host, dptr, bytes, cudaMemcpyDeviceToHost, g->stream));
  CK(cudaStreamSynchronize(g->stream));
  if (g->comm.allreduce(g->comm.ctx, g->xp_host, count, dtype, op) != 0) {
    g->poisoned = true;
    return fail(g, IGK_ENCCL, "all-reduce callback failed");
  }
  CK(cudaMemcpyAsync(dptr, g->xp_host, bytes, cudaMemcpyHostToDevice, g->stream));
  return IGK_OK;
}
// all-reduce (sum) of host values through the device scratch
igk_status xp_sum_host(igk_graph* g, long long* vals, int n) {
  if (!g->sharded) return IGK_OK;
  if (n > kXpWords) return fail(g, IGK_EINVAL, "xp_sum_host: too many values");
  CK(cudaMemcpyAsync(g->d_xp, vals, n * 8, cudaMemcpyHostToDevice, g->stream));
  igk_status st = xp_allreduce(g, g->d_xp, n, XP_I64, XP_SUM);
  if (st != IGK_OK) return st;
  CK(cudaMemcpyAsync(vals, g->d_xp, n * 8, cudaMemcpyDeviceToHost, g->stream));
  CK(cudaStreamSynchronize(g->stream));
  return IGK_OK;
}

// NEXT-3 set-up (collective): allocate this rank's record buffers and
// barrier counter, exchange {pid, device, pointers, IPC handles} through the
// transport (sum of disjoint rows), map every peer: the same process ->
// direct pointers (+ peer access across devices), another process -> CUDA
// IPC.  Re-run after a vertex-capacity growth (the buffers hold n_cap).
constexpr int kBlob = 40;  // int64 words per rank
void p2p_teardown(igk_graph* g) {
  for (int q = 0; q < g->nranks && q < 8; q++) {
    if (g->p2p_ipc[q]) {
      cudaIpcCloseMemHandle(g->p2p_bufs[q][0]);
      cudaIpcCloseMemHandle(g->p2p_bars[q]);
    }
    g->p2p_ipc[q] = false;
    g->p2p_bufs[q][0] = g->p2p_bufs[q][1] = nullptr;
    g->p2p_bars[q] = nullptr;
  }
}
// the CUB scratch of the canonical pending-list sort, sized for n_cap keys
// once (at create / growth, both collective): no allocation -- and no
// implicit device synchronisation -- between the last collective of a
// refine and its persistent round kernel (ranks may share a GPU)
igk_status sort_scratch(igk_graph* g) {
  size_t need = 0;
  cub::DeviceRadixSort::SortKeys(nullptr, need, (const uint32_t*)g->d.psi[0], (uint32_t*)g->d.psi[1],
                                 (int)std::min<long long>(g->d.n_cap, INT32_MAX), 0, g->d.idbits, g->stream);
  if (need <= g->sort_tmp_cap) return IGK_OK;
  if (g->sort_tmp) cudaFree(g->sort_tmp);
  g->sort_tmp = nullptr;
  g->sort_tmp_cap = 0;
  CK(cudaMalloc(&g->sort_tmp, need));
  g->sort_tmp_cap = need;
  return IGK_OK;
}

igk_status p2p_setup(igk_graph* g) {
  const int n = g->nranks, me = g->rank;
  if (n > 8) return fail(g, IGK_EINVAL, "p2p: at most 8 ranks");
  p2p_teardown(g);
  long long sync1 = 0;
  igk_status st = xp_sum_host(g, &sync1, 1);  // every rank closed its mappings of the old buffers
  if (st != IGK_OK) return st;
  if (g->p2p_mem) cudaFree(g->p2p_mem);
  if (g->p2p_bar) cudaFree(g->p2p_bar);
  g->p2p_mem = nullptr;
  g->p2p_bar = nullptr;
  const long long cap = g->d.n_cap;
  CK(cudaMalloc(&g->p2p_mem, (size_t)cap * 2 * sizeof(int4)));
  CK(cudaMalloc(&g->p2p_bar, 256));
  CK(cudaMemsetAsync(g->p2p_mem, 0, (size_t)cap * 2 * sizeof(int4), g->stream));
  CK(cudaMemsetAsync(g->p2p_bar, 0, 256, g->stream));
  CK(cudaStreamSynchronize(g->stream));
  g->p2p_cap = cap;
  g->p2p_rounds = 0;
  std::vector<long long> blob((size_t)n * kBlob, 0);
  long long* row = &blob[(size_t)me * kBlob];
  row[0] = (long long)getpid();
  row[1] = g->device;
  row[2] = (long long)(uintptr_t)g->p2p_mem;
  row[3] = (long long)(uintptr_t)g->p2p_bar;
  cudaIpcMemHandle_t hm{}, hb{};  // for peers in other processes (not needed inside one process)
  static_assert(sizeof(cudaIpcMemHandle_t) == 64, "IPC handle size");
  if (cudaIpcGetMemHandle(&hm, g->p2p_mem) == cudaSuccess && cudaIpcGetMemHandle(&hb, g->p2p_bar) == cudaSuccess) {
    row[20] = 1;
    std::memcpy(&row[4], &hm, 64);
    std::memcpy(&row[12], &hb, 64);
  }
  cudaGetLastError();
  st = xp_sum_host(g, blob.data(), n * kBlob);  // every rank's row (disjoint: the sum is a gather)
  if (st != IGK_OK) return st;
  for (int q = 0; q < n; q++) {
    const long long* r = &blob[(size_t)q * kBlob];
    int4* mem = nullptr;
    unsigned long long* bar = nullptr;
    if (q == me) {
      mem = g->p2p_mem;
      bar = g->p2p_bar;
    } else if (r[0] == (long long)getpid()) {  // same process: the pointers are valid here
      mem = (int4*)(uintptr_t)r[2];
      bar = (unsigned long long*)(uintptr_t)r[3];
      if ((int)r[1] != g->device) {
        cudaError_t e = cudaDeviceEnablePeerAccess((int)r[1], 0);
        if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled) CK(e);
        cudaGetLastError();
      }
    } else {  // another process: CUDA IPC (NVLink peer mapping across GPUs)
      if (!r[20]) return fail(g, IGK_ENCCL, "p2p: a peer in another process exported no IPC handle");
      cudaIpcMemHandle_t h1, h2;
      std::memcpy(&h1, &r[4], 64);
      std::memcpy(&h2, &r[12], 64);
      void* p1 = nullptr;
      void* p2 = nullptr;
      CK(cudaIpcOpenMemHandle(&p1, h1, cudaIpcMemLazyEnablePeerAccess));
      CK(cudaIpcOpenMemHandle(&p2, h2, cudaIpcMemLazyEnablePeerAccess));
      mem = (int4*)p1;
      bar = (unsigned long long*)p2;
      g->p2p_ipc[q] = true;
    }
    g->p2p_bufs[q][0] = mem;
    g->p2p_bufs[q][1] = mem + cap;
    g->p2p_bars[q] = bar;
  }
  long long sync2 = 0;
  return xp_sum_host(g, &sync2, 1);  // every rank mapped every peer before any kernel runs
}

igk_status launch_recount(igk_graph* g) {
  CK(cudaMemsetAsync(g->d_red, 0, sizeof(long long) * 262, g->stream));
  long long n = g->h_ctl->n_total;
  CK(cudaEventRecord(g->ev[4], g->stream));
  if (g->recount_tma == 1 && !g->d.adjw) {
    k_recount_tma<<<g->recount_tma_blocks, kRcT, sizeof(RcSmem), g->stream>>>(g->d, n, g->d_red, g->d_red + 1,
                                                                             g->d_red + 257);
  } else if (g->recount_tma == 2) {
    k_recount<<<g->recount_blocks, 256, 0, g->stream>>>(g->d, n, g->d_red, g->d_red + 1, g->d_red + 257);
  } else {
    // pieces of the heavy vertices go to the vertex-deletion scratch (idle
    // outside k_apply): (n_cap + slot_cap / 8) int2 >= slot_cap / 16 int4,
    // more than the <= slot_cap / 205 pieces a store can need
    Dev dd = g->d;
    long long* out_cut = g->d_red;
    long long* out_wp = g->d_red + 1;
    long long* out_cnt = g->d_red + 257;
    unsigned long long* ctr = reinterpret_cast<unsigned long long*>(g->d_red + 259);
    int4* pieces = reinterpret_cast<int4*>(g->d.vdch);
    void* args[] = {&dd, &n, &out_cut, &out_wp, &out_cnt, &ctr, &pieces};
    const void* fn = g->d.adjw ? (const void*)k_recount3<true> : (const void*)k_recount3<false>;
    CK(cudaLaunchCooperativeKernel(fn, g->d.adjw ? g->recount3w_blocks : g->recount3_blocks, kR3Threads, args, 0,
                                   g->stream));
  }
  g->launches++;
  CK(cudaGetLastError());
  CK(cudaEventRecord(g->ev[5], g->stream));
  return IGK_OK;
}

igk_status sync_ctl(igk_graph* g, int which) {
  g->ms_pending = 0;  // the stream is synchronised below: every event is complete
  // lean readback: only the output block at the head of Ctl (full copy when debugging)
  const size_t bytes = (g->debug_phases || g->check) ? sizeof(Ctl) : offsetof(Ctl, Wp);
  CK(cudaMemcpyAsync(g->h_ctl, g->d.ctl, bytes, cudaMemcpyDeviceToHost, g->stream));
  CK(cudaStreamSynchronize(g->stream));
  if (which >= 0 && g->debug_phases) {
    auto& v = g->ph[which];
    v.clear();
    for (int i = 0; i < std::min(g->h_ctl->nph, 128); i++) v.push_back({g->h_ctl->idph[i], g->h_ctl->tph[i]});
  }
  return IGK_OK;
}

// replace *p (count_old elements of `elem` bytes) by a fresh allocation of
// count_new elements: old content copied, the tail filled with byte `fill`
bool regrow(igk_graph* g, void** p, size_t elem, size_t count_old, size_t count_new, int fill) {
  void* q = nullptr;
  if (cudaMalloc(&q, std::max<size_t>(count_new, 1) * elem) != cudaSuccess) return false;
  if (*p && count_old) cudaMemcpyAsync(q, *p, count_old * elem, cudaMemcpyDeviceToDevice, g->stream);
  if (count_new > count_old) cudaMemsetAsync((char*)q + count_old * elem, fill, (count_new - count_old) * elem, g->stream);
  for (auto& a : g->allocs)
    if (a == *p) a = q;
  if (*p) {
    cudaStreamSynchronize(g->stream);
    cudaFree(*p);
  }
  *p = q;
  return true;
}

// grow every per-vertex array to new_cap vertex IDs (contents kept)
igk_status grow_vertex_capacity(igk_graph* g, long long new_cap) {
  Dev& d = g->d;
  const size_t o = (size_t)d.n_cap, n = (size_t)new_cap;
  struct A {
    void** p;
    size_t elem;
    int fill;
  } arrs[] = {
      {(void**)&d.vr, sizeof(VRec), 0},                                                        {(void**)&d.capv, 4, 0},
      {(void**)&d.active, 1, 0},   {(void**)&d.part, 1, kDel}, {(void**)&d.markA, 4, 0},  {(void**)&d.markT, 4, 0},
      {(void**)&d.markD, 4, 0},    {(void**)&d.markG, 4, 0},   {(void**)&d.markF, 4, 0},  {(void**)&d.markH, 4, 0},
      {(void**)&d.vcnt, 4, 0},     {(void**)&d.icnt, 4, 0},    {(void**)&d.Alist, 4, 0},  {(void**)&d.psi[0], 4, 0},
      {(void**)&d.psi[1], 4, 0},   {(void**)&d.psi[2], 4, 0},  {(void**)&d.cand, 4, 0},   {(void**)&d.cand2, 4, 0},
      {(void**)&d.Nlist, 4, 0},    {(void**)&d.glist, 4, 0},   {(void**)&d.rlist, 4, 0},  {(void**)&d.r3list, 8, 0},
      {(void**)&d.reloc, 8, 0},    {(void**)&d.tgt, 1, 0},     {(void**)&d.gain, 4, 0},   {(void**)&d.pw, 4, 0},
      {(void**)&d.meta, 4, 0},     {(void**)&d.metav, 4, 0},   {(void**)&d.oldp, 1, 0},   {(void**)&d.hubA, 4, 0},
      {(void**)&d.hubC, 4, 0},     {(void**)&d.hubN, 4, 0},    {(void**)&d.hubC2, 4, 0},  {(void**)&d.hubP, 4, 0},
      {(void**)&g->d_out, 4, 0},   {(void**)&d.delta, 8, 0},
  };
  for (auto& a : arrs)
    if (!regrow(g, a.p, a.elem, o, n, a.fill)) return fail(g, IGK_ENOMEM, "vertex capacity growth failed");
  if (d.vw && !regrow(g, (void**)&d.vw, 4, o, n, 0)) return fail(g, IGK_ENOMEM, "vertex capacity growth failed");
  if (d.bm && (!regrow(g, (void**)&d.bm, 8, o / 64 + 2, n / 64 + 2, 0) || !regrow(g, (void**)&d.lossbuf, 4, o, n, 0) ||
               !regrow(g, (void**)&d.recs, 16, o, n, 0)))
    return fail(g, IGK_ENOMEM, "vertex capacity growth failed");
  const size_t vdo = o + (size_t)(d.slot_cap / kVdC) + 1024, vdn = n + (size_t)(d.slot_cap / kVdC) + 1024;
  if (!regrow(g, (void**)&d.vdch, 8, 0, vdn, 0)) return fail(g, IGK_ENOMEM, "vertex capacity growth failed");
  (void)vdo;
  d.n_cap = new_cap;
  int ib = 1;
  while ((1ll << ib) < d.n_cap) ib++;
  d.idbits = ib;
  CK(cudaStreamSynchronize(g->stream));
  g->n_grow++;
  if (g->sharded) {
    igk_status st = sort_scratch(g);
    if (st != IGK_OK) return st;
  }
  if (g->p2p) return p2p_setup(g);  // the record buffers hold n_cap entries (collective: growth is)
  return IGK_OK;
}

// compact the slab into fresh arrays; live entries only.  The new capacity
// keeps at least half of it free AND room for `extra` more slots (the demand
// of the batch whose validation ran out of slots), so one compaction always
// suffices for that batch.
igk_status compact_slab(igk_graph* g, long long extra) {
  Dev& d = g->d;
  const long long n = g->h_ctl->n_total;
  std::vector<int32_t> ldeg((size_t)std::max<long long>(n, 1));
  std::vector<uint8_t> act((size_t)std::max<long long>(n, 1));
  if (n) {
    CK(vr_get(ldeg.data(), d.vr, offsetof(VRec, ldeg), 4, n, cudaMemcpyDeviceToHost, g->stream));
    CK(cudaMemcpyAsync(act.data(), d.active, n, cudaMemcpyDeviceToHost, g->stream));
    CK(cudaStreamSynchronize(g->stream));
  }
  std::vector<int64_t> noff((size_t)std::max<long long>(n, 1));
  std::vector<int32_t> ncap((size_t)std::max<long long>(n, 1));
  long long used = 0;
  for (long long v = 0; v < n; v++) {
    long long dg = act[v] ? ldeg[v] : 0;
    ldeg[v] = (int32_t)dg;  // deleted vertices keep no prefix
    long long c = act[v] ? ((dg + std::max<long long>(d.slack_min, dg / 4) + 3) & ~3ll) : 0;
    noff[v] = used;
    ncap[v] = (int32_t)c;
    used += c;
  }
  long long cap = d.slot_cap;
  while (cap < 2 * used + (1ll << 20) || cap < used + extra + (1ll << 20)) cap *= 2;  // half free + the batch
  cap = std::min<long long>(cap, (1ll << 31) - 2);
  if (used > cap) return fail(g, IGK_ENOMEM, "adjacency slab cannot hold the graph");
  int32_t *nadj = nullptr, *nadjw = nullptr, *ntwin = nullptr, *fwd = nullptr;
  int64_t* d_noff = nullptr;
  const long long old_top = g->h_ctl->slab_top;
  bool ok = cudaMalloc(&nadj, cap * 4) == cudaSuccess && cudaMalloc(&ntwin, cap * 4) == cudaSuccess &&
            (!d.adjw || cudaMalloc(&nadjw, cap * 4) == cudaSuccess) &&
            cudaMalloc(&fwd, std::max<long long>(old_top, 1) * 4) == cudaSuccess &&
            cudaMalloc(&d_noff, std::max<long long>(n, 1) * 8) == cudaSuccess;
  if (!ok) {
    cudaFree(nadj); cudaFree(ntwin); cudaFree(nadjw); cudaFree(fwd); cudaFree(d_noff);
    return fail(g, IGK_ENOMEM, "slab compaction: allocation failed");
  }
  CK(cudaMemsetAsync(nadj, 0xff, cap * 4, g->stream));
  if (nadjw) CK(cudaMemsetAsync(nadjw, 0, cap * 4, g->stream));
  if (n) CK(cudaMemcpyAsync(d_noff, noff.data(), n * 8, cudaMemcpyHostToDevice, g->stream));
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, g->device);
  k_compact_copy<<<sms * 8, 256, 0, g->stream>>>(d, n, d_noff, nadj, nadjw, ntwin, fwd);
  k_compact_twins<<<sms * 8, 256, 0, g->stream>>>(used, nadj, ntwin, fwd);
  g->launches += 2;
  CK(cudaGetLastError());
  if (n) {
    CK(vr_put(d.vr, offsetof(VRec, off), d_noff, 8, n, cudaMemcpyDeviceToDevice, g->stream));
    CK(cudaMemcpyAsync(d.capv, ncap.data(), n * 4, cudaMemcpyHostToDevice, g->stream));
    CK(vr_put(d.vr, offsetof(VRec, deg), ldeg.data(), 4, n, cudaMemcpyHostToDevice, g->stream));  // no tombstones left
    CK(vr_put(d.vr, offsetof(VRec, ldeg), ldeg.data(), 4, n, cudaMemcpyHostToDevice, g->stream));
  }
  CK(cudaStreamSynchronize(g->stream));
  int32_t* olds[3] = {d.adj, d.twin, d.adjw};
  int32_t* news[3] = {nadj, ntwin, nadjw};
  for (int i = 0; i < 3; i++) {
    if (!olds[i]) continue;
    for (auto& a : g->allocs)
      if (a == olds[i]) a = news[i];
    cudaFree(olds[i]);
  }
  d.adj = nadj;
  d.twin = ntwin;
  d.adjw = nadjw;
  cudaFree(fwd);
  cudaFree(d_noff);
  // the vertex-deletion chunk list is sized by the slab: regrow it
  if (!regrow(g, (void**)&d.vdch, 8, 0, (size_t)d.n_cap + (size_t)(cap / kVdC) + 1024, 0))
    return fail(g, IGK_ENOMEM, "slab compaction: allocation failed");
  d.slot_cap = cap;
  g->h_ctl->slab_top = used;
  CK(cudaMemcpyAsync(&d.ctl->slab_top, &g->h_ctl->slab_top, 8, cudaMemcpyHostToDevice, g->stream));
  CK(cudaStreamSynchronize(g->stream));
  g->compactions++;
  return IGK_OK;
}

// CSR checks (no self loops, no duplicates, IDs in range, weights in
// range, symmetric with equal weights) and the twin of every entry: the
// position of u in row x for the entry u -> x
bool csr_twins(int64_t n, const int64_t* xadj, const int32_t* adjncy, const int32_t* adjwgt,
               std::vector<int32_t>& twin_pos, long long ew_max = kEwMax) {
  const long long m2 = n > 0 ? xadj[n] : 0;
  std::vector<std::pair<int32_t, int32_t>> rows((size_t)m2);
  for (int64_t u = 0; u < n; u++) {
    for (int64_t j = xadj[u]; j < xadj[u + 1]; j++) {
      int32_t x = adjncy[j], w = adjwgt ? adjwgt[j] : 1;
      if (x < 0 || x >= n || x == u || w < 1 || w > ew_max) return false;
      rows[j] = {x, (int32_t)(j - xadj[u])};
    }
    std::sort(rows.begin() + xadj[u], rows.begin() + xadj[u + 1]);
    for (int64_t j = xadj[u] + 1; j < xadj[u + 1]; j++)
      if (rows[j].first == rows[j - 1].first) return false;
  }
  twin_pos.assign((size_t)std::max<long long>(m2, 1), 0);
  for (int64_t u = 0; u < n; u++) {
    for (int64_t j = xadj[u]; j < xadj[u + 1]; j++) {
      int32_t x = adjncy[j];
      auto b = rows.begin() + xadj[x], e = rows.begin() + xadj[x + 1];
      auto it = std::lower_bound(b, e, std::make_pair((int32_t)u, INT32_MIN));
      if (it == e || it->first != u) return false;
      if (adjwgt && adjwgt[xadj[x] + it->second] != adjwgt[j]) return false;
      twin_pos[j] = it->second;
    }
  }
  return true;
}

}  // namespace

extern "C" {

igk_status igk_create(const igk_options* opt, int64_t n, const int64_t* xadj, const int32_t* adjncy,
                      const int32_t* vwgt, const int32_t* adjwgt, int32_t k, double epsilon,
                      const int32_t* init_part, igk_graph** out) {
  if (!out) return IGK_EINVAL;
  *out = nullptr;
  if (n < 0 || n > kNMax || k < 2 || k > kMaxK || !(epsilon > 0.0) || !(epsilon <= 1.0)) return IGK_EINVAL;
  if (n > 0 && (!xadj || !init_part || (xadj[n] > 0 && !adjncy))) return IGK_EINVAL;
  igk_options o{};
  if (opt) o = *opt;
  const int nranks = o.nranks > 1 ? o.nranks : 1;
  const bool sharded = nranks > 1 || o.nccl_id || o.comm;  // one rank + a transport: the protocol on one GPU
  if (sharded && (o.rank < 0 || o.rank >= nranks || (!o.nccl_id && (!o.comm || !o.comm->allreduce))))
    return IGK_EINVAL;
  // ---- host-side validation of the CSR (create-time plumbing) ----
  if (n > 0 && xadj[0] != 0) return IGK_EINVAL;
  for (int64_t u = 0; u < n; u++) {
    if (xadj[u + 1] < xadj[u] || xadj[u + 1] - xadj[u] > kDegMax) return IGK_EINVAL;
    if (init_part[u] < 0 || init_part[u] >= k) return IGK_EINVAL;
    if (vwgt && (vwgt[u] < 1 || (!o.wide_weights && vwgt[u] > kVwMax))) return IGK_EINVAL;
  }
  const long long ew_max = o.wide_weights ? INT32_MAX : kEwMax;
  std::vector<int32_t> twin_pos;
  if (!csr_twins(n, xadj, adjncy, adjwgt, twin_pos, ew_max)) return IGK_EINVAL;
  if (o.wide_weights) {  // every per-vertex sum of the refine must stay exact in 32 bits
    long long tv = 0, te = 0;
    for (int64_t u = 0; u < n; u++) tv += vwgt ? vwgt[u] : 1;
    for (int64_t j = 0; j < (n > 0 ? xadj[n] : 0); j++) te += adjwgt ? adjwgt[j] : 1;
    if (tv > INT32_MAX || te / 2 > INT32_MAX || sharded) return IGK_EINVAL;
  }
  // sharded: keep the entries u -> x with owner(u) == rank or owner(x) ==
  // rank (own vertices in full + the ghost prefixes pointing at them); the
  // condition is symmetric, so the kept CSR is again symmetric
  std::vector<int64_t> fx;
  std::vector<int32_t> fa, fw;
  const long long sh_blk = nranks > 1 ? std::max<long long>(1, (n + nranks - 1) / nranks) : 1;
  if (nranks > 1) {
    auto owns = [&](long long v) { return v / sh_blk == o.rank; };
    fx.assign((size_t)n + 1, 0);
    for (int64_t u = 0; u < n; u++) {
      for (int64_t j = xadj[u]; j < xadj[u + 1]; j++)
        if (owns(u) || owns(adjncy[j])) {
          fa.push_back(adjncy[j]);
          if (adjwgt) fw.push_back(adjwgt[j]);
        }
      fx[u + 1] = (int64_t)fa.size();
    }
    xadj = fx.data();
    adjncy = fa.data();
    if (adjwgt) adjwgt = fw.data();
    if (!csr_twins(n, xadj, adjncy, adjwgt, twin_pos, ew_max)) return IGK_EINVAL;
  }
  const long long m2 = n > 0 ? xadj[n] : 0;
  igk_graph* g = new igk_graph();
  g->wide = o.wide_weights != 0;
  g->nranks = nranks;
  g->rank = nranks > 1 ? o.rank : 0;
  g->sharded = sharded;
  if (sharded && !o.nccl_id) g->comm = *o.comm;
  g->device = o.device;
  g->stream = (cudaStream_t)o.stream;
  g->e_ppm = llround(epsilon * 1e6);
  g->vw_unit = vwgt == nullptr;
  g->ew_unit = adjwgt == nullptr;
  g->check = o.check_invariants;
  DevGuard dev_guard(g->device);
  NvtxRange nv("igk_create");
  {
    int cur = -1;
    if (cudaGetDevice(&cur) != cudaSuccess || cur != g->device) {
      delete g;
      return IGK_ECUDA;
    }
  }
  {  // k_recount: 48 registers, 5 blocks of 256 per SM (measured best:
     // profiles/r01_s15_recount_ab.txt), computed per handle and device
    int sms = 0, occ = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, g->device);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_recount, 256, 0);
    g->recount_blocks = sms * std::max(1, std::min(occ, 5));
    cudaFuncSetAttribute(k_recount_tma, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(RcSmem));
    occ = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_recount_tma, kRcT, sizeof(RcSmem));
    g->recount_tma_blocks = sms * std::max(1, occ);
    // the TMA-pipelined variant is opt-in: measured 2-4x slower than the
    // direct gathers on C2 / C4 / C5 (profiles/r02_s9_recount_ab.txt)
    const char* rc = getenv("IGK_RECOUNT");
    g->recount_tma = !rc ? 0 : std::strcmp(rc, "tma") == 0 ? 1 : std::strcmp(rc, "gather") == 0 ? 2 : 0;
    int o3 = 0, o3w = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o3, k_recount3<false>, kR3Threads, 0);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o3w, k_recount3<true>, kR3Threads, 0);
    g->recount3_blocks = sms * std::max(1, o3);
    g->recount3w_blocks = sms * std::max(1, o3w);
  }
  Dev& d = g->d;
  d.k = k;
  d.n_cap = o.max_vertices > 0 ? o.max_vertices : 2 * n + 65536;
  if (d.n_cap < n || d.n_cap > kNMax) {
    delete g;
    return IGK_EINVAL;
  }
  d.slack_min = o.slack_min > 0 ? o.slack_min : 2;
  int ib = 1;
  while ((1ll << ib) < d.n_cap) ib++;
  d.idbits = ib;
  d.nranks = nranks;
  d.rank = g->rank;
  d.sharded = sharded;
  d.sh_n0 = n;
  d.sh_blk = sh_blk;
  // slack capacities and offsets (prefix sum on the host at create time)
  std::vector<int64_t> off((size_t)std::max<int64_t>(n, 1));
  std::vector<int32_t> deg((size_t)std::max<int64_t>(n, 1)), capv((size_t)std::max<int64_t>(n, 1));
  long long used = 0;
  for (int64_t u = 0; u < n; u++) {
    long long dg = xadj[u + 1] - xadj[u];
    long long c = dg + std::max<long long>(d.slack_min, dg / 4);
    c = (c + 3) & ~3ll;
    off[u] = used;
    deg[u] = (int32_t)dg;
    capv[u] = (int32_t)c;
    used += c;
  }
  d.slot_cap = o.max_slots > 0 ? o.max_slots : 4 * used + (1ll << 22);
  d.slot_cap = std::min<long long>(d.slot_cap, (1ll << 31) - 2);  // slots are int32 (twin pointers)
  if (d.slot_cap < used) {
    delete g;
    return IGK_EINVAL;
  }
  const size_t N = (size_t)d.n_cap;
  bool ok = dalloc(g, &d.vr, N) && dalloc(g, &d.capv, N) &&
            dalloc(g, &d.adj, (size_t)d.slot_cap) && dalloc(g, &d.twin, (size_t)d.slot_cap) &&
            (g->ew_unit || dalloc(g, &d.adjw, (size_t)d.slot_cap)) &&
            dalloc(g, &d.active, N) && (g->vw_unit || dalloc(g, &d.vw, N)) && dalloc(g, &d.part, N) &&
            dalloc(g, &d.markA, N) && dalloc(g, &d.markT, N) && dalloc(g, &d.markD, N) &&
            dalloc(g, &d.markG, N) && dalloc(g, &d.vcnt, N) && dalloc(g, &d.icnt, N) &&
            dalloc(g, &d.Alist, N) && dalloc(g, &d.psi[0], N) && dalloc(g, &d.psi[1], N) &&
            dalloc(g, &d.psi[2], N) && dalloc(g, &d.cand, N) && dalloc(g, &d.cand2, N) &&
            dalloc(g, &d.vdch, N + (size_t)(d.slot_cap / kVdC) + 1024) && dalloc(g, &d.markF, N) && dalloc(g, &d.oldp, N) && dalloc(g, &d.markH, N) &&
            dalloc(g, &d.hubA, N) && dalloc(g, &d.hubC, N) && dalloc(g, &d.hubN, N) && dalloc(g, &d.hubC2, N) &&
            dalloc(g, &d.hubP, N) && dalloc(g, &d.Nlist, N) && dalloc(g, &d.glist, N) &&
            dalloc(g, &d.rlist, N) && dalloc(g, &d.r3list, N) && dalloc(g, &d.reloc, N) &&
            dalloc(g, &d.tgt, N) && dalloc(g, &d.gain, N) && dalloc(g, &d.pw, N) && dalloc(g, &d.meta, N) && dalloc(g, &d.metav, N) &&
            dalloc(g, &d.hist0, 256 * kDigits) && dalloc(g, &d.histR, 3 * 256 * kDigits) &&
            dalloc(g, &d.blkcnt, 4096) && dalloc(g, &d.ctl, 1) && dalloc(g, &g->d_out, N) && dalloc(g, &d.delta, N) &&
            dalloc(g, &g->d_red, 262) && dalloc(g, &g->d_xp, kXpWords);
  if (ok && sharded)  // sharded exchange buffers (bitmap words, restoration keys, round records)
    ok = dalloc(g, &d.bm, N / 64 + 2) && dalloc(g, &d.lossbuf, N) && dalloc(g, &d.recs, N);
  if (!ok) {
    igk_destroy(g);
    return IGK_ENOMEM;
  }
  if (sharded) {
    cudaMemsetAsync(d.bm, 0, (N / 64 + 2) * 8, g->stream);
    if (o.nccl_id) {  // the library's own communicator over NVLink / NVSwitch
      const NcclApi* api = nccl_api();
      ncclUniqueId id;
      std::memcpy(&id, o.nccl_id, sizeof id);
      ncclComm_t comm = nullptr;
      if (!api || api->init_rank(&comm, nranks, id, g->rank) != ncclSuccess) {
        igk_destroy(g);
        return IGK_ENCCL;
      }
      g->nccl = comm;
    }
  }
  g->p2p = sharded && o.p2p;
  g->fallback_ppm = sharded || g->wide ? 0 : std::max<long long>(0, o.fgp_fallback_ppm);
  g->n_at_full = n;
  g->ranks_per_device = o.ranks_per_device > 1 ? o.ranks_per_device : 1;
  if (cudaMallocHost(&g->h_ctl, sizeof(Ctl)) != cudaSuccess ||
      cudaHostAlloc(&g->h_map, sizeof(Ctl), cudaHostAllocMapped) != cudaSuccess ||
      cudaHostAlloc(&g->h_flag, 64, cudaHostAllocMapped) != cudaSuccess ||
      cudaHostGetDevicePointer((void**)&d.hmap, g->h_map, 0) != cudaSuccess ||
      cudaHostGetDevicePointer((void**)&d.hflag, g->h_flag, 0) != cudaSuccess) {
    igk_destroy(g);
    return IGK_ENOMEM;
  }
  *g->h_flag = 0;
  d.seq = 0;
  for (auto& e : g->ev) cudaEventCreate(&e);
  for (auto& e : g->ev_stage) cudaEventCreateWithFlags(&e, cudaEventDisableTiming);
  // zero-init
  cudaStream_t s = g->stream;
  cudaMemsetAsync(d.active, 0, N, s);
  cudaMemsetAsync(d.part, kDel, N, s);
  cudaMemsetAsync(d.vr, 0, N * sizeof(VRec), s);
  cudaMemsetAsync(d.capv, 0, N * 4, s);
  cudaMemsetAsync(d.markA, 0, N * 4, s);
  cudaMemsetAsync(d.markT, 0, N * 4, s);
  cudaMemsetAsync(d.markD, 0, N * 4, s);
  cudaMemsetAsync(d.markG, 0, N * 4, s);
  cudaMemsetAsync(d.markF, 0, N * 4, s);
  cudaMemsetAsync(d.markH, 0, N * 4, s);
  cudaMemsetAsync(d.vcnt, 0, N * 4, s);
  cudaMemsetAsync(d.icnt, 0, N * 4, s);
  cudaMemsetAsync(d.hist0, 0, 256 * kDigits * 8, s);
  // the slab: every slot a tombstone until written (the recount reads whole
  // int4 chunks of a prefix; the slack slots it masks are then initialised)
  cudaMemsetAsync(d.adj, 0xff, (size_t)d.slot_cap * 4, s);
  cudaMemsetAsync(d.oldp, kPsi, N, s);  // saved labels: read (masked) for every neighbour by the commit
  if (d.adjw) cudaMemsetAsync(d.adjw, 0, (size_t)d.slot_cap * 4, s);
  cudaMemsetAsync(d.histR, 0, 3 * 256 * kDigits * 8, s);
  cudaMemsetAsync(d.ctl, 0, sizeof(Ctl), s);
  // upload
  int64_t* d_xadj = nullptr;
  int32_t *d_adjncy = nullptr, *d_adjwgt = nullptr;
  if (cudaMalloc(&d_xadj, (n + 1) * 8) != cudaSuccess || cudaMalloc(&d_adjncy, std::max<long long>(m2, 1) * 4) != cudaSuccess ||
      (!g->ew_unit && cudaMalloc(&d_adjwgt, std::max<long long>(m2, 1) * 4) != cudaSuccess)) {
    cudaFree(d_xadj);
    cudaFree(d_adjncy);
    igk_destroy(g);
    return IGK_ENOMEM;
  }
  std::vector<int32_t> twin_h((size_t)std::max<long long>(used, 1));
  for (int64_t u = 0; u < n; u++)
    for (int64_t j = xadj[u]; j < xadj[u + 1]; j++) {
      int32_t x = adjncy[j];
      twin_h[off[u] + (j - xadj[u])] = (int32_t)(off[x] + twin_pos[j]);
    }
  std::vector<int32_t>().swap(twin_pos);
  std::vector<uint8_t> part8((size_t)std::max<int64_t>(n, 1)), act((size_t)std::max<int64_t>(n, 1), 1);
  for (int64_t u = 0; u < n; u++) part8[u] = (uint8_t)init_part[u];
  cudaError_t e = cudaSuccess;
  // every upload is ordered on the handle's stream after the zero-fills
  // above (the stream may be a non-blocking one)
  const auto H2D = cudaMemcpyHostToDevice;
  if (n > 0) {
    e = cudaMemcpyAsync(d_xadj, xadj, (n + 1) * 8, H2D, s);
    if (e == cudaSuccess && m2) e = cudaMemcpyAsync(d_adjncy, adjncy, m2 * 4, H2D, s);
    if (e == cudaSuccess && m2 && d_adjwgt) e = cudaMemcpyAsync(d_adjwgt, adjwgt, m2 * 4, H2D, s);
    if (e == cudaSuccess) e = vr_put(d.vr, offsetof(VRec, off), off.data(), 8, n, H2D, s);
    if (e == cudaSuccess && used) e = cudaMemcpyAsync(d.twin, twin_h.data(), used * 4, H2D, s);
    if (e == cudaSuccess) e = vr_put(d.vr, offsetof(VRec, deg), deg.data(), 4, n, H2D, s);
    if (e == cudaSuccess) e = vr_put(d.vr, offsetof(VRec, ldeg), deg.data(), 4, n, H2D, s);
    if (e == cudaSuccess) e = cudaMemcpyAsync(d.capv, capv.data(), n * 4, H2D, s);
    if (e == cudaSuccess) e = cudaMemcpyAsync(d.part, part8.data(), n, H2D, s);
    if (e == cudaSuccess) e = cudaMemcpyAsync(d.active, act.data(), n, H2D, s);
    if (e == cudaSuccess && d.vw) e = cudaMemcpyAsync(d.vw, vwgt, n * 4, H2D, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  }
  if (e == cudaSuccess && n > 0) {
    k_build<<<1184, 256, 0, s>>>(d, d_xadj, d_adjncy, d_adjwgt, n);
    g->launches++;
    e = cudaGetLastError();
  }
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  cudaFree(d_xadj);
  cudaFree(d_adjncy);
  cudaFree(d_adjwgt);
  if (e != cudaSuccess) {
    igk_destroy(g);
    return IGK_ECUDA;
  }
  // control block: n_total, slab top, W, W_p, cut (from the reduction kernel)
  long long W = 0;
  for (int64_t u = 0; u < n; u++) W += vwgt ? vwgt[u] : 1;
  std::memset(g->h_ctl, 0, sizeof(Ctl));
  g->h_ctl->n_total = n;
  g->h_ctl->slab_top = used;
  g->h_ctl->W = W;
  g->h_ctl->err_idx = kNoErr;
  if (launch_recount(g) != IGK_OK) {
    igk_destroy(g);
    return IGK_ECUDA;
  }
  long long red[257];
  if (cudaMemcpyAsync(red, g->d_red, sizeof(red), cudaMemcpyDeviceToHost, s) != cudaSuccess ||
      cudaStreamSynchronize(s) != cudaSuccess) {
    igk_destroy(g);
    return IGK_ECUDA;
  }
  g->h_ctl->cut = red[0];  // sharded: this rank's partial (edges whose smaller endpoint it owns)
  g->cut_total = red[0];
  if (sharded && xp_sum_host(g, &g->cut_total, 1) != IGK_OK) {
    igk_destroy(g);
    return IGK_ENCCL;
  }
  for (int p = 0; p < k; p++) g->h_ctl->Wp[p] = red[1 + p];
  if (cudaMemcpyAsync(d.ctl, g->h_ctl, sizeof(Ctl), cudaMemcpyHostToDevice, s) != cudaSuccess ||
      cudaStreamSynchronize(s) != cudaSuccess) {
    igk_destroy(g);
    return IGK_ECUDA;
  }
  g->debug_phases = getenv("IGK_DEBUG_PHASES") != nullptr || getenv("IGK_DEBUG_ARRIVALS") != nullptr;
  // opt-in per-CTA barrier arrival stamps (tools/phase_profile.py)
  if (getenv("IGK_DEBUG_ARRIVALS")) {
    if (!dalloc(g, &d.dbg, 128 * 4096)) {
      igk_destroy(g);
      return IGK_ENOMEM;
    }
    cudaMemsetAsync(d.dbg, 0, 128 * 4096 * 8, s);
    cudaStreamSynchronize(s);
  }
  // persistent grids
  g->smem_refine = sizeof(RefSmem);
  g->smem_step = sizeof(StepSmem);
  cudaFuncSetAttribute(k_refine, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)g->smem_refine);
  cudaFuncSetAttribute(k_refine_sh, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)g->smem_refine);
  cudaFuncSetAttribute(k_step, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)g->smem_step);
  const int dv = g->device;
  g->grid_apply = coop_grid((const void*)k_apply, 0, o.blocks_per_sm, dv);
  g->grid_refine = coop_grid((const void*)k_refine, g->smem_refine, o.blocks_per_sm, dv);
  g->grid_refine = std::min(g->grid_refine, coop_grid((const void*)k_step, g->smem_step, o.blocks_per_sm, dv));
  g->grid_refine = std::min(g->grid_refine, coop_grid((const void*)k_refine_sh, g->smem_refine, o.blocks_per_sm, dv));
  if (g->grid_apply > 4096) g->grid_apply = 4096;
  {  // k_refine may run wider than the fused k_step (A/B: IGK_REFINE_BPS)
    const char* e = getenv("IGK_REFINE_BPS");
    const int bps = e ? atoi(e) : o.blocks_per_sm;
    g->grid_refine_k = std::min(4096, coop_grid((const void*)k_refine, g->smem_refine, bps, dv));
  }
  g->grid_apply_wide = std::min(4096, coop_grid((const void*)k_apply, 0, 64, dv));

  g->split_b = kSplitB;
  if (const char* e = getenv("IGK_SPLIT_B")) g->split_b = atoll(e);
  g->epochA = next_epoch(g);
  if (sharded && sort_scratch(g) != IGK_OK) {
    igk_destroy(g);
    return IGK_ENOMEM;
  }
  if (g->p2p) {
    cudaFuncSetAttribute(k_rounds_p2p, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)g->smem_refine);
    const int gp = coop_grid((const void*)k_rounds_p2p, g->smem_refine, 1, dv);
    g->grid_p2p = std::max(1, gp / g->ranks_per_device);
    const igk_status ps = p2p_setup(g);
    if (ps != IGK_OK) {
      t_create_err = "p2p set-up: " + g->err;
      igk_destroy(g);
      return ps;
    }
  }
  *out = g;
  return IGK_OK;
}

static ApplyArgs make_apply_args(igk_graph* g, const int4* dm, int64_t count);
static RefineArgs make_refine_args(igk_graph* g, int after_apply, int global = 0);

// capacity of the per-batch scratch (hash, new IDs)
static igk_status prepare_apply(igk_graph* g, int64_t count) {
  // duplicate-detection hash: >= 2 * count slots, power of two
  long long need = 64;
  while (need < 2 * count + 2) need <<= 1;
  if (need > g->hash_cap) {
    if (g->d.hkeys) cudaFree(g->d.hkeys);
    if (g->d.hcnt) cudaFree(g->d.hcnt);
    g->d.hkeys = nullptr;
    g->d.hcnt = nullptr;
    if (cudaMalloc(&g->d.hkeys, need * 8) != cudaSuccess || cudaMalloc(&g->d.hcnt, need * 4) != cudaSuccess)
      return fail(g, IGK_ENOMEM, "hash allocation failed");
    g->hash_cap = need;
    CK(cudaMemsetAsync(g->d.hkeys, 0xff, need * 8, g->stream));  // empty; kept empty by k_apply
    CK(cudaMemsetAsync(g->d.hcnt, 0, need * 4, g->stream));
  }
  if (count > g->newid_cap) {
    if (g->d.newid) cudaFree(g->d.newid);
    g->d.newid = nullptr;
    g->newid_cap = 0;
    long long cap = grow_cap(count);
    if (cudaMalloc(&g->d.newid, cap * 4) != cudaSuccess) return fail(g, IGK_ENOMEM, "newid allocation failed");
    g->newid_cap = cap;
  }
  g->d.hmask = g->hash_cap - 1;
  return IGK_OK;
}

// launch of k_apply alone (no host synchronisation)
static igk_status launch_apply(igk_graph* g, const int4* dm, int64_t count) {
  igk_status st = prepare_apply(g, count);
  if (st != IGK_OK) return st;
  ApplyArgs a = make_apply_args(g, dm, count);
  void* args[] = {(void*)&g->d, (void*)&a};
  CK(cudaEventRecord(g->ev[2], g->stream));
  CK(cudaLaunchCooperativeKernel((const void*)k_apply, g->grid_apply, kThreads, args, 0, g->stream));
  g->launches++;
  CK(cudaEventRecord(g->ev[3], g->stream));
  return IGK_OK;
}

// after the control block was read back: apply status
static igk_status finish_apply(igk_graph* g, int64_t* bad_index) {
  cudaEventElapsedTime(&g->ms_apply, g->ev[2], g->ev[3]);
  if (g->h_ctl->err_idx != kNoErr) {
    if (bad_index) *bad_index = g->h_ctl->err_idx;
    char buf[128];
    snprintf(buf, sizeof buf, "invalid modifier at index %lld", g->h_ctl->err_idx);
    return fail(g, IGK_EINVAL, buf);
  }
  if (g->h_ctl->err_nomem) return fail(g, IGK_ENOMEM, "vertex or slot capacity exhausted");
  g->refine_due = true;
  return IGK_OK;
}

static ApplyArgs make_apply_args(igk_graph* g, const int4* dm, int64_t count) {
  ApplyArgs a;
  a.mods = dm;
  a.B = count;
  a.n0 = g->h_ctl->n_total;
  a.epD = next_epoch(g);
  a.epT = next_epoch(g);
  a.epG = next_epoch(g);
  a.epA = g->epochA;
  a.vw_unit = g->vw_unit;
  a.ew_unit = g->ew_unit;
  a.phases = 3;
  return a;
}

static RefineArgs make_refine_args(igk_graph* g, int after_apply, int global) {
  RefineArgs a;
  a.e_ppm = g->e_ppm;
  a.epC1 = next_epoch(g);
  a.epN = next_epoch(g);
  a.epC2 = next_epoch(g);
  a.epF = next_epoch(g);
  a.epE = next_epoch(g);
  a.epA = g->epochA;
  a.after_apply = after_apply;
  a.global = global;
  a.prof = g->prof;
  if (g->prof)  // per-phase counters of THIS refine (ordered before its launch on the stream)
    cudaMemsetAsync(&g->d.ctl->phscan[0], 0, sizeof(long long) * 16, g->stream);
  return a;
}

static igk_status launch_refine_sh(igk_graph* g, const RefineArgs& a, const ShardArgs& sh) {
  void* args[] = {(void*)&g->d, (void*)&a, (void*)&sh};
  CK(cudaLaunchCooperativeKernel((const void*)k_refine_sh, g->grid_refine, kThreads, args, g->smem_refine, g->stream));
  g->launches++;
  return IGK_OK;
}

static igk_status launch_refine(igk_graph* g, int after_apply, int global = 0) {
  RefineArgs a = make_refine_args(g, after_apply, global);
  void* args[] = {(void*)&g->d, (void*)&a};
  CK(cudaEventRecord(g->ev[0], g->stream));
  CK(cudaLaunchCooperativeKernel((const void*)k_refine, g->grid_refine_k, kThreads, args, g->smem_refine,
                                 g->stream));
  g->launches++;
  CK(cudaEventRecord(g->ev[1], g->stream));
  return IGK_OK;
}

static igk_status finish_refine(igk_graph* g, igk_refine_stats* stats);

// sharded refine (collective; refine.cuh RefineMode): F0 | bitmap | F1+F2 |
// bitmap | F3 (+ R3 keys | keys | R3) | canonical pending list | per round:
// gain | records | finish | post.  All-reduces are fixed-size sums of
// disjoint contributions; the host synchronises after F3 / R3 (restoration
// decision, pending count) and after every round (pending count).
static igk_status refine_sharded(igk_graph* g, igk_refine_stats* stats) {
  RefineArgs ra = make_refine_args(g, 0);
  ShardArgs sh{};
  Dev& d = g->d;
  const long long nw = (g->h_ctl->n_total + 63) / 64;
  CK(cudaEventRecord(g->ev[0], g->stream));
  CK(cudaMemsetAsync(d.bm, 0, (size_t)std::max<long long>(nw, 1) * 8, g->stream));
  igk_status st = IGK_OK;
  auto launch = [&](int mode) {
    sh.mode = mode;
    return launch_refine_sh(g, ra, sh);
  };
  if ((st = launch(kShF0)) != IGK_OK) return st;
  if ((st = xp_allreduce(g, d.bm, nw, XP_I64, XP_SUM)) != IGK_OK) return st;  // C1 (disjoint bits: OR)
  if ((st = launch(kShF1)) != IGK_OK) return st;
  if ((st = xp_allreduce(g, d.bm, nw, XP_I64, XP_SUM)) != IGK_OK) return st;  // C2
  if ((st = launch(kShF3)) != IGK_OK) return st;
  if ((st = sync_ctl(g, -1)) != IGK_OK) return st;
  if (g->h_ctl->sh_flag) {  // restoration: the owners' keys, then the replicated select
    if ((st = xp_allreduce(g, d.lossbuf, g->h_ctl->n_total, XP_U32, XP_SUM)) != IGK_OK) return st;
    if ((st = launch(kShR3)) != IGK_OK) return st;
    if ((st = sync_ctl(g, -1)) != IGK_OK) return st;
  }
  const long long np = g->h_ctl->sh_np;
  if (np > 0) {  // the canonical pending list: psi[0] sorted by ID into psi[1]
    size_t need = g->sort_tmp_cap;  // sized for n_cap keys at create / growth (sort_scratch)
    CK(cub::DeviceRadixSort::SortKeys(g->sort_tmp, need, (const uint32_t*)d.psi[0], (uint32_t*)d.psi[1], (int)np,
                                      0, d.idbits, g->stream));
    g->launches++;
    sh.np = np;
    if (g->p2p) {  // NEXT-3: every round in one persistent kernel, records through peer memory
      P2PArgs pa{};
      pa.n = g->nranks;
      pa.self = g->rank;
      for (int q = 0; q < g->nranks; q++) {
        pa.bufs[q][0] = g->p2p_bufs[q][0];
        pa.bufs[q][1] = g->p2p_bufs[q][1];
        pa.bars[q] = g->p2p_bars[q];
      }
      pa.bar_base = (unsigned long long)g->nranks * (unsigned long long)g->p2p_rounds;
      pa.timeout = 4000000000ll;  // ~2 s at 1.9 GHz: a peer that never arrives is an error, not a hang
      long long npv = np;
      void* args[] = {(void*)&g->d, (void*)&ra, (void*)&npv, (void*)&pa};
      CK(cudaLaunchCooperativeKernel((const void*)k_rounds_p2p, g->grid_p2p, kThreads, args, g->smem_refine,
                                     g->stream));
      g->launches++;
      if ((st = sync_ctl(g, -1)) != IGK_OK) return st;
      if (g->h_ctl->p2p_err) {
        g->poisoned = true;
        return fail(g, IGK_ENCCL, "p2p rounds: a peer never reached the device barrier");
      }
      g->p2p_rounds += g->h_ctl->rs_rounds_all;  // rounds_all counted from 0 by kShF0
    } else
    for (long long r = 0; r <= np; r++) {  // <= |Psi| rounds (the minimum-ID pending vertex always moves)
      CK(cudaMemsetAsync(d.recs, 0, (size_t)np * 16, g->stream));
      if ((st = launch(kShGain)) != IGK_OK) return st;
      if ((st = xp_allreduce(g, d.recs, 4 * np, XP_U32, XP_SUM)) != IGK_OK) return st;  // records
      if ((st = launch(kShFinish)) != IGK_OK) return st;
      if ((st = sync_ctl(g, -1)) != IGK_OK) return st;
      if (g->h_ctl->rs_pending == 0) break;
    }
  }
  if ((st = launch(kShPost)) != IGK_OK) return st;
  CK(cudaEventRecord(g->ev[1], g->stream));
  if ((st = sync_ctl(g, 1)) != IGK_OK) return st;
  // the per-rank sums: affected / inserted / expanded / scanned (replicated
  // parts added by rank 0 only) and the partial cut
  long long* so = g->h_ctl->st_out;
  long long v[5] = {so[ST_AFFECTED], so[ST_INSERTED], so[ST_EXPANDED], so[ST_SCANNED], so[ST_CUT]};
  if ((st = xp_sum_host(g, v, 5)) != IGK_OK) return st;
  so[ST_AFFECTED] = v[0];
  so[ST_INSERTED] = v[1];
  so[ST_EXPANDED] = v[2];
  so[ST_SCANNED] = v[3];
  so[ST_CUT] = g->cut_total = v[4];
  return finish_refine(g, stats);
}

// after a capacity failure (detected in validation: nothing was mutated),
// grow the vertex arrays and/or compact the slab so the batch can be re-run
static igk_status make_room(igk_graph* g) {
  const int why = g->h_ctl->err_nomem;
  igk_status st = IGK_OK;
  if (why & 1) {
    long long need = g->h_ctl->n_total + g->h_ctl->n_ins;
    if (need > kNMax) return fail(g, IGK_ENOMEM, "vertex ID space (2^30) exhausted");
    st = grow_vertex_capacity(g, std::min<long long>(kNMax, std::max<long long>(2 * g->d.n_cap, need + 65536)));
  }
  // the batch's own slot demand (recorded by the rejected validation) sizes
  // the compaction, so one compaction suffices for it
  if (st == IGK_OK && (why & 2)) st = compact_slab(g, g->h_ctl->slab_need);
  return st;
}

// sharded apply (collective): validation launch, the verdict all-reduced
// (lowest invalid index: MIN; capacity flags: MAX) on the stream, mutation
// launch -- every rank rejects or applies the batch alike; a capacity
// shortfall on any rank makes every rank grow / compact and re-run it
static igk_status apply_dev_sharded(igk_graph* g, const int4* dm, int64_t count, int64_t* bad_index) {
  for (int attempt = 0;; attempt++) {
    igk_status st = prepare_apply(g, count);
    if (st != IGK_OK) return st;
    ApplyArgs a = make_apply_args(g, dm, count);
    void* args[] = {(void*)&g->d, (void*)&a};
    CK(cudaEventRecord(g->ev[2], g->stream));
    a.phases = 1;
    CK(cudaLaunchCooperativeKernel((const void*)k_apply, g->grid_apply, kThreads, args, 0, g->stream));
    st = xp_allreduce(g, &g->d.ctl->sh_err[0], 1, XP_I64, XP_MIN);
    if (st == IGK_OK) st = xp_allreduce(g, &g->d.ctl->sh_err[1], 1, XP_I64, XP_MAX);
    if (st != IGK_OK) return st;
    a.phases = 2;
    CK(cudaLaunchCooperativeKernel((const void*)k_apply, g->grid_apply, kThreads, args, 0, g->stream));
    g->launches += 2;
    CK(cudaEventRecord(g->ev[3], g->stream));
    st = sync_ctl(g, 0);
    if (st != IGK_OK) return st;
    g->h_ctl->err_idx = g->h_ctl->sh_err[0];  // the global verdict
    g->h_ctl->err_nomem = (int)g->h_ctl->sh_err[1];
    if (g->h_ctl->err_idx == kNoErr && g->h_ctl->err_nomem && attempt < 2) {
      st = make_room(g);
      if (st != IGK_OK) return st;
      continue;
    }
    st = finish_apply(g, bad_index);
    if (st != IGK_OK) return st;
    g->cut_total = g->h_ctl->cut;  // the ranks' partial cuts -> the global cut
    return xp_sum_host(g, &g->cut_total, 1);
  }
}

static igk_status apply_dev(igk_graph* g, const int4* dm, int64_t count, int64_t* first_new_id, int64_t* bad_index) {
  if (bad_index) *bad_index = -1;
  if (first_new_id) *first_new_id = g->h_ctl->n_total;
  if (count == 0) return IGK_OK;
  if (g->wide) return fail(g, IGK_EINVAL, "wide-weight handles accept no modifiers");
  if (g->sharded) return apply_dev_sharded(g, dm, count, bad_index);
  for (int attempt = 0;; attempt++) {
    igk_status st = launch_apply(g, dm, count);
    if (st != IGK_OK) return st;
    st = sync_ctl(g, 0);
    if (st != IGK_OK) return st;
    // a vertex-ID shortfall hides the slab demand of the new vertices: up to two rounds of growth
    if (g->h_ctl->err_idx == kNoErr && g->h_ctl->err_nomem && attempt < 2) {
      st = make_room(g);
      if (st != IGK_OK) return st;
      continue;
    }
    st = finish_apply(g, bad_index);
    if (st == IGK_OK) g->mods_since_full += count;
    return st;
  }
}

static igk_status prepare_apply(igk_graph* g, int64_t count);

// igk_step fast path: the kernel posts its output head into host-mapped
// memory and raises a flag (publish, common.cuh); the host polls the flag
// instead of a D2H copy + stream synchronisation.  Debug / check modes keep
// the full copy.
static bool notice_begin(igk_graph* g) {
  if (g->debug_phases || g->check) {
    g->d.seq = 0;
    return false;
  }
  if (++g->seq == 0) ++g->seq;  // 0 means "no notice"
  g->d.seq = g->seq;
  return true;
}
static igk_status notice_wait(igk_graph* g) {
  volatile unsigned* f = g->h_flag;
  for (long long i = 1; *f != g->seq; i++) {
    if ((i & 255) == 0) {  // the kernel failed or ended without a notice: fall back
      cudaError_t e = cudaStreamQuery(g->stream);
      if (e == cudaErrorNotReady) continue;
      if (e != cudaSuccess) CK(e);
      if (*f != g->seq) {
        g->n_notice_fallback++;
        return sync_ctl(g, 1);
      }
    }
  }
  std::atomic_thread_fence(std::memory_order_acquire);
  std::memcpy(g->h_ctl, (const void*)g->h_map, offsetof(Ctl, Wp));
  g->ms_pending = 1;  // ev[1] completes after the kernel exits: convert lazily
  return IGK_OK;
}

// one launch of a step (fused k_step, or k_apply + k_refine for large
// batches); *posted = the kernel posts a host-mapped completion notice
static igk_status step_launch(igk_graph* g, const int4* dm, int64_t count, bool* posted) {
  igk_status st;
  *posted = false;
  if (count == 0) {
    st = launch_refine(g, 0);
    if (st != IGK_OK) return st;
  } else if (count >= g->split_b) {
    // large batch: k_apply at full occupancy (64 registers: 2x the warps
    // of the fused kernel for its latency-bound gathers and atomics), then
    // k_refine on the same stream -- no host round trip between them; a
    // rejected batch makes the refine exit untouched (after_apply)
    st = prepare_apply(g, count);
    if (st != IGK_OK) return st;
    ApplyArgs aa = make_apply_args(g, dm, count);
    RefineArgs ra = make_refine_args(g, 1);
    void* a1[] = {(void*)&g->d, (void*)&aa};
    void* a2[] = {(void*)&g->d, (void*)&ra};
    Dev dn = g->d;  // the refine posts the completion notice, not the apply
    const bool fast = notice_begin(g);
    void* a1n[] = {(void*)&dn, (void*)&aa};
    CK(cudaEventRecord(g->ev[0], g->stream));
    CK(cudaLaunchCooperativeKernel((const void*)k_apply, g->grid_apply_wide, kThreads, fast ? a1n : a1, 0,
                                   g->stream));
    CK(cudaLaunchCooperativeKernel((const void*)k_refine, g->grid_refine_k, kThreads, a2, g->smem_refine, g->stream));
    g->d.seq = 0;
    g->launches += 2;
    g->n_split++;
    CK(cudaEventRecord(g->ev[1], g->stream));
    *posted = fast;
  } else {  // apply + refine in ONE persistent launch (k_step)
    st = prepare_apply(g, count);
    if (st != IGK_OK) return st;
    ApplyArgs aa = make_apply_args(g, dm, count);
    RefineArgs ra = make_refine_args(g, 1);
    const bool fast = notice_begin(g);
    void* args[] = {(void*)&g->d, (void*)&aa, (void*)&ra};
    CK(cudaEventRecord(g->ev[0], g->stream));
    CK(cudaLaunchCooperativeKernel((const void*)k_step, g->grid_refine, kThreads, args, g->smem_step, g->stream));
    g->d.seq = 0;
    g->launches++;
    g->n_fused++;
    CK(cudaEventRecord(g->ev[1], g->stream));
    *posted = fast;
  }
  return IGK_OK;
}

// wait for a launched step; a batch rejected only for capacity (nothing was
// mutated) is re-run after growing / compacting the store
static igk_status step_complete(igk_graph* g, const int4* dm, int64_t count, bool posted, igk_refine_stats* stats,
                                int64_t* bad_index) {
  igk_status st;
  for (int attempt = 0;; attempt++) {
    st = posted ? notice_wait(g) : sync_ctl(g, 1);
    if (st != IGK_OK) return st;
    if (count > 0 && g->h_ctl->err_idx == kNoErr && g->h_ctl->err_nomem && attempt < 2) {
      st = make_room(g);  // the kernel stopped before any mutation: grow / compact, then re-run
      if (st != IGK_OK) return st;
      st = step_launch(g, dm, count, &posted);
      if (st != IGK_OK) return st;
      continue;
    }
    break;
  }
  if (count > 0) {
    g->ms_apply = 0;  // fused: the whole step is in ms_refine
    if (g->h_ctl->err_idx != kNoErr) {
      if (bad_index) *bad_index = g->h_ctl->err_idx;
      char buf[128];
      snprintf(buf, sizeof buf, "invalid modifier at index %lld", g->h_ctl->err_idx);
      return fail(g, IGK_EINVAL, buf);  // the kernel ended before the refine: state unchanged
    }
    if (g->h_ctl->err_nomem) return fail(g, IGK_ENOMEM, "vertex or slot capacity exhausted");
    g->mods_since_full += count;
  }
  return finish_refine(g, stats);
}

static igk_status step_dev(igk_graph* g, const int4* dm, int64_t count, igk_refine_stats* stats,
                           int64_t* first_new_id, int64_t* bad_index) {
  if (bad_index) *bad_index = -1;
  if (first_new_id) *first_new_id = g->h_ctl->n_total;
  igk_status st;
  if (g->wide && count > 0) return fail(g, IGK_EINVAL, "wide-weight handles accept no modifiers");
  if (g->sharded) {  // sharded: the collective apply, then the collective refine
    st = apply_dev(g, dm, count, first_new_id, bad_index);
    if (st != IGK_OK) return st;
    return refine_sharded(g, stats);
  }
  bool posted = false;
  st = step_launch(g, dm, count, &posted);
  if (st != IGK_OK) return st;
  return step_complete(g, dm, count, posted, stats, bad_index);
}

// host batch -> g->d_mods on the handle stream.  A page-locked caller buffer
// (cudaHostAlloc / cudaHostRegister / torch pin_memory) is DMA'd directly;
// pageable memory goes through the handle's pinned staging buffer.  The copy
// is complete before the call returns (the step synchronises the stream).
static igk_status stage_batch(igk_graph* g, const igk_modifier* mods, int64_t count) {
  if (count > g->d_mods_cap) {
    if (g->d_mods) cudaFree(g->d_mods);
    g->d_mods = nullptr;
    g->d_mods_cap = 0;
    long long cap = grow_cap(count);
    if (cudaMalloc(&g->d_mods, cap * 16) != cudaSuccess) return fail(g, IGK_ENOMEM, "batch allocation failed");
    g->d_mods_cap = cap;
  }
  cudaPointerAttributes at{};
  const bool pinned = cudaPointerGetAttributes(&at, mods) == cudaSuccess && at.type == cudaMemoryTypeHost;
  cudaGetLastError();  // a pageable pointer is not an error
  if (pinned) {
    CK(cudaMemcpyAsync(g->d_mods, mods, count * 16, cudaMemcpyHostToDevice, g->stream));
    return IGK_OK;
  }
  if (count > g->h_stage_cap) {
    if (g->h_stage) cudaFreeHost(g->h_stage);
    g->h_stage = nullptr;
    g->h_stage_cap = 0;
    long long cap = grow_cap(count);
    if (cudaMallocHost(&g->h_stage, cap * sizeof(igk_modifier)) != cudaSuccess)
      return fail(g, IGK_ENOMEM, "pinned staging allocation failed");
    g->h_stage_cap = cap;
  }
  std::memcpy(g->h_stage, mods, count * sizeof(igk_modifier));
  CK(cudaMemcpyAsync(g->d_mods, g->h_stage, count * 16, cudaMemcpyHostToDevice, g->stream));
  return IGK_OK;
}

igk_status igk_apply_modifiers(igk_graph* g, const igk_modifier* mods, int64_t count, int64_t* first_new_id,
                               int64_t* bad_index) {
  if (!g || g->poisoned) return IGK_ESTATE;
  ENTRY(g, "igk_apply_modifiers");
  if (count < 0 || (count > 0 && !mods)) return fail(g, IGK_EINVAL, "bad batch pointer/count");
  if (count == 0) return apply_dev(g, nullptr, 0, first_new_id, bad_index);
  igk_status st = stage_batch(g, mods, count);
  if (st != IGK_OK) return st;
  return apply_dev(g, g->d_mods, count, first_new_id, bad_index);
}

igk_status igk_apply_modifiers_device(igk_graph* g, const igk_modifier* d_mods, int64_t count,
                                      int64_t* first_new_id, int64_t* bad_index) {
  if (!g || g->poisoned) return IGK_ESTATE;
  ENTRY(g, "igk_apply_modifiers_device");
  if (count < 0 || (count > 0 && !d_mods)) return fail(g, IGK_EINVAL, "bad batch pointer/count");
  return apply_dev(g, (const int4*)d_mods, count, first_new_id, bad_index);
}

static igk_status finish_refine(igk_graph* g, igk_refine_stats* stats) {
  if (!g->ms_pending) cudaEventElapsedTime(&g->ms_refine, g->ev[0], g->ev[1]);
  g->refine_due = false;
  g->delta_replaced = false;
  g->epochA = next_epoch(g);
  const long long* so = g->h_ctl->st_out;
  if (stats) {
    stats->affected = so[ST_AFFECTED];
    stats->inserted = so[ST_INSERTED];
    stats->expanded = so[ST_EXPANDED];
    stats->filtered_in = so[ST_FILTERED_IN];
    stats->expanded_in = so[ST_EXPANDED_IN];
    stats->evicted = so[ST_EVICTED];
    stats->rounds = so[ST_ROUNDS];
    stats->moves_applied = so[ST_MOVES_APPLIED];
    stats->moves_deferred = so[ST_MOVES_DEFERRED];
    stats->cut = so[ST_CUT];
    stats->cap = so[ST_CAP];
    stats->max_part_weight = so[ST_MAXW];
    stats->imbalanced = so[ST_IMBAL];
    stats->adj_entries_scanned = so[ST_SCANNED];
  }
  const bool imbal = so[ST_IMBAL] != 0;
  if (g->check) {  // invariant I1/I2: maintained cut and W_p equal a recount (sharded: collective)
    int64_t cut = 0;
    int64_t wp[256];
    igk_status st = igk_recount(g, &cut, wp);
    if (st != IGK_OK) return st;
    bool bad = cut != (g->sharded ? g->cut_total : g->h_ctl->cut);
    for (int p = 0; p < g->d.k; p++) bad |= wp[p] != g->h_ctl->Wp[p];
    if (bad) {
      g->poisoned = true;
      return fail(g, IGK_ESTATE, "invariant check failed: maintained cut/W_p differ from the recount");
    }
  }
  if (stats) stats->repartitioned = 0;
  // the FGP fallback policy (reading F9): modifiers since the last full
  // partition >= fgp_fallback_ppm / 1e6 of the active vertices counted then
  if (g->fallback_ppm > 0 && g->mods_since_full * 1000000ll >= g->fallback_ppm * g->n_at_full) {
    int64_t cut = 0;
    igk_status st = igk_repartition(g, 6, &cut);
    if (st != IGK_OK) return st;
    long long mx = 0;
    for (int p = 0; p < g->d.k; p++) mx = std::max(mx, g->h_ctl->Wp[p]);
    if (stats) {
      stats->repartitioned = 1;
      stats->cut = cut;
      stats->max_part_weight = mx;
      stats->imbalanced = mx > so[ST_CAP];
    }
    return mx > so[ST_CAP] ? IGK_WIMBALANCED : IGK_OK;
  }
  return imbal ? IGK_WIMBALANCED : IGK_OK;
}

igk_status igk_refine(igk_graph* g, igk_refine_stats* stats) {
  if (!g || g->poisoned) return IGK_ESTATE;
  ENTRY(g, "igk_refine");
  if (g->sharded) return refine_sharded(g, stats);
  igk_status st = launch_refine(g, 0);
  if (st != IGK_OK) return st;
  st = sync_ctl(g, 1);
  if (st != IGK_OK) return st;
  return finish_refine(g, stats);
}

igk_status igk_refine_global(igk_graph* g, igk_refine_stats* stats) {
  if (!g || g->poisoned) return IGK_ESTATE;
  ENTRY(g, "igk_refine_global");
  if (g->sharded) return fail(g, IGK_EINVAL, "igk_refine_global: single-GPU handles only");
  igk_status st = launch_refine(g, 0, 1);  // boundary scan + refine: one launch
  if (st != IGK_OK) return st;
  st = sync_ctl(g, 1);
  if (st != IGK_OK) return st;
  return finish_refine(g, stats);
}

igk_status igk_step(igk_graph* g, const igk_modifier* mods, int64_t count, igk_refine_stats* stats,
                    int64_t* first_new_id, int64_t* bad_index) {
  if (!g || g->poisoned) return IGK_ESTATE;
  ENTRY(g, "igk_step");
  if (count < 0 || (count > 0 && !mods)) return fail(g, IGK_EINVAL, "bad batch pointer/count");
  if (count > 0) {
    igk_status st = stage_batch(g, mods, count);
    if (st != IGK_OK) return st;
  }
  return step_dev(g, g->d_mods, count, stats, first_new_id, bad_index);
}

igk_status igk_step_device(igk_graph* g, const igk_modifier* d_mods, int64_t count, igk_refine_stats* stats,
                           int64_t* first_new_id, int64_t* bad_index) {
  if (!g || g->poisoned) return IGK_ESTATE;
  ENTRY(g, "igk_step_device");
  if (count < 0 || (count > 0 && !d_mods)) return fail(g, IGK_EINVAL, "bad batch pointer/count");
  return step_dev(g, (const int4*)d_mods, count, stats, first_new_id, bad_index);
}

// ---------------------------------------------------------------------------
// NEXT-2: IGK-FGP v1 full partitioning (fgp.cuh; readings F1-F6)
// ---------------------------------------------------------------------------
}  // extern "C"
namespace {
struct FgpLevel {
  long long n = 0, m2 = 0;
  int64_t* xadj = nullptr;
  int32_t *adj = nullptr, *w = nullptr, *vw = nullptr;
  int32_t* cmap = nullptr;  // vertex -> coarse vertex of the next level
};
struct DevBuf {  // frees its device allocations on scope exit
  std::vector<void*> ps;
  template <class T>
  T* get(size_t n) {
    void* p = nullptr;
    if (cudaMalloc(&p, std::max<size_t>(n, 1) * sizeof(T)) != cudaSuccess) return nullptr;
    ps.push_back(p);
    return (T*)p;
  }
  ~DevBuf() {
    for (void* p : ps) cudaFree(p);
  }
};

// one handle per level (wide weights), the global boundary refinement
// repeated while it lowers the cut (<= kFgpPasses), the refined labels out
constexpr int kFgpPasses = 8;     // F6: global refinement passes on the coarsest level
constexpr int kFgpLpPasses = 16;  // F7: label-propagation passes per finer level
igk_status fgp_refine_level(const igk_options& o, const FgpLevel& L, int k, double eps, std::vector<int32_t>& part,
                            std::string& err) {
  std::vector<int64_t> xa(L.n + 1);
  std::vector<int32_t> aj(std::max<long long>(L.m2, 1)), ww(std::max<long long>(L.m2, 1)), vw(std::max<long long>(L.n, 1));
  cudaStream_t s = (cudaStream_t)o.stream;
  if (cudaMemcpyAsync(xa.data(), L.xadj, (L.n + 1) * 8, cudaMemcpyDeviceToHost, s) != cudaSuccess ||
      (L.m2 && cudaMemcpyAsync(aj.data(), L.adj, L.m2 * 4, cudaMemcpyDeviceToHost, s) != cudaSuccess) ||
      (L.m2 && cudaMemcpyAsync(ww.data(), L.w, L.m2 * 4, cudaMemcpyDeviceToHost, s) != cudaSuccess) ||
      cudaMemcpyAsync(vw.data(), L.vw, L.n * 4, cudaMemcpyDeviceToHost, s) != cudaSuccess ||
      cudaStreamSynchronize(s) != cudaSuccess) {
    err = "fgp: level read-back failed";
    return IGK_ECUDA;
  }
  igk_options lo = o;
  lo.wide_weights = 1;
  lo.check_invariants = 0;
  lo.nranks = 0;
  lo.nccl_id = nullptr;
  lo.comm = nullptr;
  lo.p2p = 0;
  igk_graph* h = nullptr;
  const bool trace = getenv("IGK_FGP_TRACE") != nullptr;
  auto now = [] { return std::chrono::steady_clock::now(); };
  auto ms = [](auto a, auto b) { return std::chrono::duration<double, std::milli>(b - a).count(); };
  auto t0 = now();
  igk_status st = igk_create(&lo, L.n, xa.data(), aj.data(), vw.data(), ww.data(), k, eps, part.data(), &h);
  auto t1 = now();
  if (st != IGK_OK) {
    err = std::string("fgp: level handle: ") + igk_last_error(nullptr);
    return st;
  }
  long long prev = -1;
  for (int p = 0; p < kFgpPasses; p++) {
    igk_refine_stats rs{};
    st = igk_refine_global(h, &rs);
    if (st != IGK_OK && st != IGK_WIMBALANCED) break;
    st = IGK_OK;
    if (trace) fprintf(stderr, "fgp n=%lld pass %d cut %lld rounds %lld moves %lld t=%.2f ms\n", L.n, p, (long long)rs.cut,
                       (long long)rs.rounds, (long long)rs.moves_applied, ms(t1, now()));
    if (prev >= 0 && rs.cut >= prev) break;
    prev = rs.cut;
  }
  if (trace) fprintf(stderr, "fgp n=%lld m2=%lld create %.2f ms refine %.2f ms\n", L.n, L.m2, ms(t0, t1), ms(t1, now()));
  if (st == IGK_OK) st = igk_partition(h, part.data(), (int64_t)part.size(), nullptr);
  if (st != IGK_OK) err = std::string("fgp: level refine: ") + igk_last_error(h);
  igk_destroy(h);
  return st;
}
}  // namespace
extern "C" {

// the multilevel core on a device CSR (L[0]; weights explicit): coarsening
// F1-F4, initial partition F5, coarsest refinement F6, label propagation F7.
// *d_part_out (from mem) gets the partition of L[0].
static igk_status fgp_core(const igk_options& o, DevBuf& mem, std::vector<FgpLevel>& L, long long Wt, int k,
                           double epsilon, int group_size, int32_t** d_part_out, std::string& err) {
  cudaStream_t s = (cudaStream_t)o.stream;
  const long long n = L[0].n;
  const int kMaxLv = 32;
  int* d_cnt = mem.get<int>(4);
  unsigned long long* d_ecnt = mem.get<unsigned long long>(1);
  if (!d_cnt || !d_ecnt) return IGK_ENOMEM;
  auto fail_cuda = [&]() { return IGK_ECUDA; };
  const int grid = 1184, blk = 256;
  // ---- coarsening (readings F1-F4) ----
  while ((int)L.size() - 1 < kMaxLv && L.back().n >= 35ll * k) {
    FgpLevel& G = L.back();
    const long long nl = G.n;
    int32_t* sel = mem.get<int32_t>(nl);
    int32_t* P = mem.get<int32_t>(nl);
    int32_t* Q = mem.get<int32_t>(nl);
    int32_t* label = mem.get<int32_t>(nl);
    unsigned long long* key = mem.get<unsigned long long>(nl);
    unsigned long long* skey = mem.get<unsigned long long>(nl);
    int32_t* val = mem.get<int32_t>(nl);
    int32_t* sval = mem.get<int32_t>(nl);
    long long* mark = mem.get<long long>(nl);
    long long* segstart = mem.get<long long>(nl);
    int32_t* flag = mem.get<int32_t>(nl);
    int32_t* gid = mem.get<int32_t>(nl);
    int32_t* cmap = mem.get<int32_t>(nl);
    if (!sel || !P || !Q || !label || !key || !skey || !val || !sval || !mark || !segstart || !flag || !gid || !cmap)
      return IGK_ENOMEM;
    k_fgp_select<<<grid, blk, 0, s>>>(nl, G.xadj, G.adj, G.w, sel);
    cudaMemsetAsync(d_cnt, 0, 12, s);
    cudaMemsetAsync(d_cnt + 3, 0x7f, 4, s);  // iso0 = "none" (0x7f7f7f7f > any ID)
    k_fgp_iso<<<grid, blk, 0, s>>>(nl, sel, d_cnt + 3);
    k_fgp_roots<<<grid, blk, 0, s>>>(nl, sel, d_cnt + 3, P, label, d_cnt);
    int left = 0;
    if (cudaMemcpyAsync(&left, d_cnt, 4, cudaMemcpyDeviceToHost, s) != cudaSuccess ||
        cudaStreamSynchronize(s) != cudaSuccess)
      return fail_cuda();
    for (int t = 1; left > 0 && t < 64; t++) {  // synchronous pointer jumping (F2)
      cudaMemsetAsync(d_cnt, 0, 4, s);
      k_fgp_jump<<<grid, blk, 0, s>>>(nl, P, Q, label, t, d_cnt);
      std::swap(P, Q);
      if (cudaMemcpyAsync(&left, d_cnt, 4, cudaMemcpyDeviceToHost, s) != cudaSuccess ||
          cudaStreamSynchronize(s) != cudaSuccess)
        return fail_cuda();
    }
    // (root, label) stable radix sort of the vertex IDs (F3)
    k_fgp_keys<<<grid, blk, 0, s>>>(nl, P, label, key, val);
    int ib = 1;
    while ((1ll << ib) < nl) ib++;
    size_t tb = 0;
    cub::DeviceRadixSort::SortPairs(nullptr, tb, key, skey, val, sval, (int)nl, 0, ib + 8, s);
    void* tmp = mem.get<char>(tb);
    if (!tmp) return IGK_ENOMEM;
    cub::DeviceRadixSort::SortPairs(tmp, tb, key, skey, val, sval, (int)nl, 0, ib + 8, s);
    k_fgp_segmark<<<grid, blk, 0, s>>>(nl, skey, mark);
    size_t tb2 = 0;
    cub::DeviceScan::InclusiveScan(nullptr, tb2, mark, segstart, cuda::maximum<>(), (int)nl, s);
    void* tmp2 = mem.get<char>(tb2);
    if (!tmp2) return IGK_ENOMEM;
    cub::DeviceScan::InclusiveScan(tmp2, tb2, mark, segstart, cuda::maximum<>(), (int)nl, s);
    k_fgp_groups<<<grid, blk, 0, s>>>(nl, segstart, group_size, flag);
    size_t tb3 = 0;  // gid[i] = the number of group starts up to i (group index + 1)
    cub::DeviceScan::InclusiveSum(nullptr, tb3, flag, gid, (int)nl, s);
    void* tmp3 = mem.get<char>(tb3);
    if (!tmp3) return IGK_ENOMEM;
    cub::DeviceScan::InclusiveSum(tmp3, tb3, flag, gid, (int)nl, s);
    k_fgp_cmap<<<grid, blk, 0, s>>>(nl, flag, gid, sval, cmap, d_cnt + 1);
    int hv[2] = {0, 0};
    int lastgid = 0;
    if (cudaMemcpyAsync(hv, d_cnt, 8, cudaMemcpyDeviceToHost, s) != cudaSuccess ||
        cudaMemcpyAsync(&lastgid, gid + nl - 1, 4, cudaMemcpyDeviceToHost, s) != cudaSuccess ||
        cudaStreamSynchronize(s) != cudaSuccess)
      return fail_cuda();
    const long long nc = lastgid, coarsenable = nl - hv[1];
    if (coarsenable * 10 < nl * 9 || nc >= nl) break;  // F4: fewer than 90% coarsenable / no progress
    // contraction
    FgpLevel C;
    C.n = nc;
    C.vw = mem.get<int32_t>(nc);
    C.xadj = mem.get<int64_t>(nc + 1);
    unsigned long long* ekey = mem.get<unsigned long long>(G.m2);
    unsigned long long* sekey = mem.get<unsigned long long>(G.m2);
    int32_t* ew = mem.get<int32_t>(G.m2);
    int32_t* sew = mem.get<int32_t>(G.m2);
    unsigned long long* ukey = mem.get<unsigned long long>(G.m2);
    int32_t* uw = mem.get<int32_t>(G.m2);
    int* d_nu = mem.get<int>(1);
    int64_t* rowcnt = mem.get<int64_t>(nc + 1);
    if (!C.vw || !C.xadj || !ekey || !sekey || !ew || !sew || !ukey || !uw || !d_nu || !rowcnt) return IGK_ENOMEM;
    cudaMemsetAsync(C.vw, 0, nc * 4, s);
    k_fgp_cvw<<<grid, blk, 0, s>>>(nl, cmap, G.vw, C.vw);
    cudaMemsetAsync(d_ecnt, 0, 8, s);
    k_fgp_edges<<<grid, blk, 0, s>>>(nl, G.xadj, G.adj, G.w, cmap, ekey, ew, d_ecnt);
    unsigned long long ne = 0;
    if (cudaMemcpyAsync(&ne, d_ecnt, 8, cudaMemcpyDeviceToHost, s) != cudaSuccess ||
        cudaStreamSynchronize(s) != cudaSuccess)
      return fail_cuda();
    int cb = 1;
    while ((1ll << cb) < nc) cb++;
    size_t tb4 = 0;
    cub::DeviceRadixSort::SortPairs(nullptr, tb4, ekey, sekey, ew, sew, (int)ne, 0, 32 + cb, s);
    size_t tb5 = 0;
    cub::DeviceReduce::ReduceByKey(nullptr, tb5, sekey, ukey, sew, uw, d_nu, cuda::std::plus<>(), (int)ne, s);
    void* tmp4 = mem.get<char>(std::max(tb4, tb5));
    if (!tmp4) return IGK_ENOMEM;
    if (ne) {
      cub::DeviceRadixSort::SortPairs(tmp4, tb4, ekey, sekey, ew, sew, (int)ne, 0, 32 + cb, s);
      cub::DeviceReduce::ReduceByKey(tmp4, tb5, sekey, ukey, sew, uw, d_nu, cuda::std::plus<>(), (int)ne, s);
    } else {
      cudaMemsetAsync(d_nu, 0, 4, s);
    }
    int nu = 0;
    if (cudaMemcpyAsync(&nu, d_nu, 4, cudaMemcpyDeviceToHost, s) != cudaSuccess ||
        cudaStreamSynchronize(s) != cudaSuccess)
      return fail_cuda();
    C.m2 = nu;
    C.adj = mem.get<int32_t>(nu);
    C.w = uw;  // the reduced weights, already in (row, column) order
    if (!C.adj) return IGK_ENOMEM;
    cudaMemsetAsync(rowcnt, 0, (nc + 1) * 8, s);
    k_fgp_rowcount<<<grid, blk, 0, s>>>(nu, ukey, rowcnt + 1);
    k_fgp_rows<<<grid, blk, 0, s>>>(nu, ukey, C.adj);
    size_t tb6 = 0;
    cub::DeviceScan::InclusiveSum(nullptr, tb6, rowcnt, C.xadj, (int)(nc + 1), s);
    void* tmp6 = mem.get<char>(tb6);
    if (!tmp6) return IGK_ENOMEM;
    cub::DeviceScan::InclusiveSum(tmp6, tb6, rowcnt, C.xadj, (int)(nc + 1), s);
    if (cudaGetLastError() != cudaSuccess) return fail_cuda();
    G.cmap = cmap;
    L.push_back(C);
  }
  const int nl = (int)L.size() - 1;
  // ---- initial partition of the coarsest graph (F5) + global refinement (F6) ----
  std::vector<int32_t> part((size_t)L[nl].n);
  int32_t* dpart = mem.get<int32_t>(n);  // n = L[0].n  // the partition of the current level (n_l <= n)
  int32_t* dtmp = mem.get<int32_t>(n);
  {
    uint8_t* vis = mem.get<uint8_t>(L[nl].n);
    int32_t* queue = mem.get<int32_t>(L[nl].n);
    if (!dpart || !dtmp || !vis || !queue) return IGK_ENOMEM;
    k_fgp_initial<<<1, 1, 0, s>>>(L[nl].n, L[nl].xadj, L[nl].adj, L[nl].vw, k, dpart, vis, queue);
    if (cudaMemcpyAsync(part.data(), dpart, L[nl].n * 4, cudaMemcpyDeviceToHost, s) != cudaSuccess ||
        cudaStreamSynchronize(s) != cudaSuccess)
      return fail_cuda();
  }
  igk_status st = fgp_refine_level(o, L[nl], k, epsilon, part, err);
  if (st != IGK_OK) return st;
  if (cudaMemcpyAsync(dpart, part.data(), L[nl].n * 4, cudaMemcpyHostToDevice, s) != cudaSuccess) return fail_cuda();
  // ---- projection + label propagation at every finer level (F7) ----
  if (nl > 0) {
    const long long cap = cap_of(Wt, llround(epsilon * 1e6), k);
    const long long nmax = L[0].n;
    int32_t* tgt = mem.get<int32_t>(nmax);
    int32_t* gain = mem.get<int32_t>(nmax);
    int32_t* flag = mem.get<int32_t>(nmax);
    int32_t* ids = mem.get<int32_t>(nmax);
    int32_t* sel = mem.get<int32_t>(nmax);
    int32_t* sid = mem.get<int32_t>(nmax);
    unsigned long long* key = mem.get<unsigned long long>(nmax);
    unsigned long long* skey = mem.get<unsigned long long>(nmax);
    long long* wts = mem.get<long long>(nmax);
    long long* incl = mem.get<long long>(nmax);
    long long* mark = mem.get<long long>(nmax);
    long long* segs = mem.get<long long>(nmax);
    unsigned long long* W = mem.get<unsigned long long>(k);
    long long* dW = mem.get<long long>(k);
    int* d_nm = mem.get<int>(1);
    unsigned long long* d_mv = mem.get<unsigned long long>(2);
    if (!tgt || !gain || !flag || !ids || !sel || !sid || !key || !skey || !wts || !incl || !mark || !segs || !W ||
        !dW || !d_nm || !d_mv)
      return IGK_ENOMEM;
    // CUB scratch sized for the finest level
    size_t t1 = 0, t2 = 0, t3 = 0, t4 = 0;
    cub::DeviceSelect::Flagged(nullptr, t1, ids, flag, sel, d_nm, (int)nmax, s);
    cub::DeviceRadixSort::SortPairs(nullptr, t2, key, skey, sel, sid, (int)nmax, 0, 39, s);
    cub::DeviceScan::InclusiveSum(nullptr, t3, wts, incl, (int)nmax, s);
    cub::DeviceScan::InclusiveScan(nullptr, t4, mark, segs, cuda::maximum<>(), (int)nmax, s);
    size_t tb = std::max(std::max(t1, t2), std::max(t3, t4));
    void* tmp = mem.get<char>(tb);
    if (!tmp) return IGK_ENOMEM;
    k_lp_iota<<<grid, blk, 0, s>>>(nmax, ids);
    for (int l = nl - 1; l >= 0; l--) {
      const FgpLevel& F = L[l];
      const int nlv = (int)F.n;
      k_fgp_project<<<grid, blk, 0, s>>>(F.n, F.cmap, dpart, dtmp);
      std::swap(dpart, dtmp);
      cudaMemsetAsync(W, 0, k * 8, s);
      cudaMemsetAsync(dW, 0, k * 8, s);
      k_lp_pw<<<grid, blk, 0, s>>>(F.n, dpart, F.vw, W);
      for (int pass = 0; pass < kFgpLpPasses; pass++) {
        cudaMemsetAsync(d_mv, 0, 16, s);
        k_lp_gain<<<grid, kLpThreads, 0, s>>>(F.n, F.xadj, F.adj, F.w, dpart, k, tgt, gain);
        k_lp_filter<<<grid, blk, 0, s>>>(F.n, F.xadj, F.adj, tgt, gain, flag);
        size_t tb1 = tb;
        cub::DeviceSelect::Flagged(tmp, tb1, ids, flag, sel, d_nm, nlv, s);
        int nm = 0;
        if (cudaMemcpyAsync(&nm, d_nm, 4, cudaMemcpyDeviceToHost, s) != cudaSuccess ||
            cudaStreamSynchronize(s) != cudaSuccess)
          return fail_cuda();
        if (nm == 0) break;
        k_lp_keys<<<grid, blk, 0, s>>>(d_nm, sel, tgt, gain, key);
        size_t tb2 = tb;
        cub::DeviceRadixSort::SortPairs(tmp, tb2, key, skey, sel, sid, nm, 0, 39, s);
        k_lp_segs<<<grid, blk, 0, s>>>(d_nm, skey, sid, F.vw, wts, mark);
        size_t tb3 = tb;
        cub::DeviceScan::InclusiveSum(tmp, tb3, wts, incl, nm, s);
        size_t tb4 = tb;
        cub::DeviceScan::InclusiveScan(tmp, tb4, mark, segs, cuda::maximum<>(), nm, s);
        k_lp_admit<<<grid, blk, 0, s>>>(d_nm, skey, sid, incl, segs, W, cap, F.vw, gain, dpart, dW, d_mv);
        k_lp_applyw<<<1, 256, 0, s>>>(k, W, dW);
        unsigned long long mv[2] = {0, 0};
        if (cudaMemcpyAsync(mv, d_mv, 16, cudaMemcpyDeviceToHost, s) != cudaSuccess ||
            cudaStreamSynchronize(s) != cudaSuccess)
          return fail_cuda();
        if (getenv("IGK_FGP_TRACE"))
          fprintf(stderr, "fgp lp n=%lld pass %d survivors %d moved %llu dcut %llu\n", F.n, pass, nm, mv[0], mv[1]);
        if (mv[0] == 0) break;
      }
    }
    if (cudaGetLastError() != cudaSuccess) return fail_cuda();
  }
  *d_part_out = dpart;
  return IGK_OK;
}


igk_status igk_fgp_partition(const igk_options* opt, int64_t n, const int64_t* xadj, const int32_t* adjncy,
                             const int32_t* vwgt, const int32_t* adjwgt, int32_t k, double epsilon,
                             int32_t group_size, int32_t* part_out, int64_t* level_n, int32_t* nlevels) {
  if (n < 1 || !xadj || !part_out || k < 2 || k > kMaxK || group_size < 2 || !(epsilon > 0.0) ||
      !(epsilon <= 1.0) || n > kNMax)
    return IGK_EINVAL;
  igk_options o{};
  if (opt) o = *opt;
  DevGuard dev_guard(o.device);
  NvtxRange nv("igk_fgp_partition");
  std::vector<int32_t> twin_pos;
  if (xadj[0] != 0 || !csr_twins(n, xadj, adjncy, adjwgt, twin_pos, INT32_MAX)) return IGK_EINVAL;
  std::vector<int32_t>().swap(twin_pos);
  {  // coarse weights are int32: both totals must fit (F4)
    long long tv = 0, te = 0;
    for (int64_t v = 0; v < n; v++) tv += vwgt ? vwgt[v] : 1;
    for (int64_t j = 0; j < xadj[n]; j++) te += adjwgt ? adjwgt[j] : 1;
    if (tv > INT32_MAX || te > INT32_MAX) return IGK_EINVAL;
    if (vwgt)
      for (int64_t v = 0; v < n; v++)
        if (vwgt[v] < 0) return IGK_EINVAL;
  }
  cudaStream_t s = (cudaStream_t)o.stream;
  DevBuf mem;
  std::vector<FgpLevel> L(1);
  const long long m2 = xadj[n];
  L[0].n = n;
  L[0].m2 = m2;
  L[0].xadj = mem.get<int64_t>(n + 1);
  L[0].adj = mem.get<int32_t>(m2);
  L[0].w = mem.get<int32_t>(m2);
  L[0].vw = mem.get<int32_t>(n);
  if (!L[0].xadj || !L[0].adj || !L[0].w || !L[0].vw) return IGK_ENOMEM;
  {
    std::vector<int32_t> w1, v1;
    if (!adjwgt) w1.assign((size_t)std::max<long long>(m2, 1), 1);
    if (!vwgt) v1.assign((size_t)n, 1);
    if (cudaMemcpyAsync(L[0].xadj, xadj, (n + 1) * 8, cudaMemcpyHostToDevice, s) != cudaSuccess ||
        (m2 && cudaMemcpyAsync(L[0].adj, adjncy, m2 * 4, cudaMemcpyHostToDevice, s) != cudaSuccess) ||
        (m2 && cudaMemcpyAsync(L[0].w, adjwgt ? adjwgt : w1.data(), m2 * 4, cudaMemcpyHostToDevice, s) != cudaSuccess) ||
        cudaMemcpyAsync(L[0].vw, vwgt ? vwgt : v1.data(), n * 4, cudaMemcpyHostToDevice, s) != cudaSuccess ||
        cudaStreamSynchronize(s) != cudaSuccess)
      return IGK_ECUDA;
  }
  long long Wt = 0;
  for (int64_t v = 0; v < n; v++) Wt += vwgt ? vwgt[v] : 1;
  int32_t* dpart = nullptr;
  std::string err;
  igk_status st = fgp_core(o, mem, L, Wt, k, epsilon, group_size, &dpart, err);
  if (st != IGK_OK) {
    t_create_err = err.empty() ? "igk_fgp_partition: device failure" : err;
    return st;
  }
  if (nlevels) *nlevels = (int32_t)L.size();
  if (level_n)
    for (size_t l = 0; l < L.size(); l++) level_n[l] = L[l].n;
  if (cudaMemcpyAsync(part_out, dpart, n * 4, cudaMemcpyDeviceToHost, s) != cudaSuccess ||
      cudaStreamSynchronize(s) != cudaSuccess)
    return IGK_ECUDA;
  return IGK_OK;
}

igk_status igk_repartition(igk_graph* g, int32_t group_size, int64_t* out_cut) {
  if (!g || g->poisoned) return IGK_ESTATE;
  ENTRY(g, "igk_repartition");
  if (g->sharded || g->wide) return fail(g, IGK_EINVAL, "igk_repartition: single-GPU, narrow-weight handles only");
  if (group_size < 2) return fail(g, IGK_EINVAL, "igk_repartition: group_size < 2");
  if (g->refine_due) return fail(g, IGK_ESTATE, "igk_repartition: a batch was applied and not yet refined");
  cudaStream_t s = g->stream;
  Dev& d = g->d;
  const long long n = g->h_ctl->n_total;
  DevBuf mem;
  int32_t* act = mem.get<int32_t>(n + 1);
  int32_t* did = mem.get<int32_t>(n + 1);
  int* d_cnt = mem.get<int>(1);
  if (!act || !did || !d_cnt) return fail(g, IGK_ENOMEM, "igk_repartition: allocation failed");
  cudaMemsetAsync(d_cnt, 0, 4, s);
  cudaMemsetAsync(act + n, 0, 4, s);
  k_rp_flag<<<1184, 256, 0, s>>>(d, n, act, d_cnt);
  size_t tb = 0;
  cub::DeviceScan::ExclusiveSum(nullptr, tb, act, did, (int)(n + 1), s);
  void* tmp = mem.get<char>(tb);
  if (!tmp) return fail(g, IGK_ENOMEM, "igk_repartition: allocation failed");
  cub::DeviceScan::ExclusiveSum(tmp, tb, act, did, (int)(n + 1), s);
  int hv[2] = {0, 0};
  CK(cudaMemcpyAsync(&hv[0], d_cnt, 4, cudaMemcpyDeviceToHost, s));
  CK(cudaMemcpyAsync(&hv[1], did + n, 4, cudaMemcpyDeviceToHost, s));
  CK(cudaStreamSynchronize(s));
  if (hv[0]) return fail(g, IGK_ESTATE, "igk_repartition: pending (pseudo-partition) vertices");
  const long long na = hv[1];
  if (na < 1) return fail(g, IGK_EINVAL, "igk_repartition: no active vertex");
  std::vector<FgpLevel> L(1);
  FgpLevel& L0 = L[0];
  L0.n = na;
  long long* cdeg = mem.get<long long>(na + 1);
  L0.xadj = mem.get<int64_t>(na + 1);
  L0.vw = mem.get<int32_t>(na);
  if (!cdeg || !L0.xadj || !L0.vw) return fail(g, IGK_ENOMEM, "igk_repartition: allocation failed");
  cudaMemsetAsync(cdeg, 0, (na + 1) * 8, s);
  k_rp_deg<<<1184, 256, 0, s>>>(d, n, act, did, cdeg, L0.vw);
  size_t tb2 = 0;
  cub::DeviceScan::ExclusiveSum(nullptr, tb2, cdeg, (long long*)L0.xadj, (int)(na + 1), s);
  void* tmp2 = mem.get<char>(tb2);
  if (!tmp2) return fail(g, IGK_ENOMEM, "igk_repartition: allocation failed");
  cub::DeviceScan::ExclusiveSum(tmp2, tb2, cdeg, (long long*)L0.xadj, (int)(na + 1), s);
  long long m2 = 0;
  CK(cudaMemcpyAsync(&m2, L0.xadj + na, 8, cudaMemcpyDeviceToHost, s));
  CK(cudaStreamSynchronize(s));
  L0.m2 = m2;
  int32_t* radj = mem.get<int32_t>(m2);
  int32_t* rw = mem.get<int32_t>(m2);
  L0.adj = mem.get<int32_t>(m2);
  L0.w = mem.get<int32_t>(m2);
  if (!radj || !rw || !L0.adj || !L0.w) return fail(g, IGK_ENOMEM, "igk_repartition: allocation failed");
  k_rp_rows<<<1184, 256, 0, s>>>(d, n, act, did, (const long long*)L0.xadj, radj, rw);
  if (m2 > 0) {  // rows in ascending neighbour order (the BFS of F5 walks rows in order)
    size_t tb3 = 0;
    cub::DeviceSegmentedSort::SortPairs(nullptr, tb3, radj, L0.adj, rw, L0.w, (int)m2, (int)na, L0.xadj, L0.xadj + 1, s);
    void* tmp3 = mem.get<char>(tb3);
    if (!tmp3) return fail(g, IGK_ENOMEM, "igk_repartition: allocation failed");
    cub::DeviceSegmentedSort::SortPairs(tmp3, tb3, radj, L0.adj, rw, L0.w, (int)m2, (int)na, L0.xadj, L0.xadj + 1, s);
  }
  g->launches += 5;
  CK(cudaGetLastError());
  // both totals must fit the int32 coarse weights (F4); W is maintained
  const long long Wt = g->h_ctl->W;
  if (Wt > INT32_MAX || (long long)m2 * (g->ew_unit ? 1 : 255) > INT32_MAX)
    return fail(g, IGK_EINVAL, "igk_repartition: total weights exceed the FGP's int32 range");
  igk_options o{};
  o.device = g->device;
  o.stream = (void*)s;
  int32_t* dpart = nullptr;
  std::string err;
  igk_status st = fgp_core(o, mem, L, Wt, d.k, (double)g->e_ppm / 1e6, group_size, &dpart, err);
  if (st != IGK_OK) return fail(g, st, err.empty() ? "igk_repartition: FGP failed" : err.c_str());
  k_rp_install<<<1184, 256, 0, s>>>(d, n, act, did, dpart);
  g->launches++;
  // maintained cut and W_p from the reduction kernel
  st = launch_recount(g);
  if (st != IGK_OK) return st;
  long long red[259];
  CK(cudaMemcpyAsync(red, g->d_red, sizeof(red), cudaMemcpyDeviceToHost, s));
  CK(cudaStreamSynchronize(s));
  g->h_ctl->cut = red[0];
  for (int p = 0; p < d.k; p++) g->h_ctl->Wp[p] = red[1 + p];
  g->h_ctl->n_delta = 0;
  CK(cudaMemcpyAsync(&d.ctl->cut, &g->h_ctl->cut, 8, cudaMemcpyHostToDevice, s));
  CK(cudaMemcpyAsync(&d.ctl->Wp[0], &g->h_ctl->Wp[0], 8 * d.k, cudaMemcpyHostToDevice, s));
  CK(cudaMemcpyAsync(&d.ctl->n_delta, &g->h_ctl->n_delta, 4, cudaMemcpyHostToDevice, s));
  CK(cudaStreamSynchronize(s));
  g->delta_replaced = true;
  g->mods_since_full = 0;
  g->n_at_full = na;
  if (out_cut) *out_cut = red[0];
  return IGK_OK;
}

igk_status igk_stage_batch(igk_graph* g, const igk_modifier* mods, int64_t count) {
  if (!g || g->poisoned) return IGK_ESTATE;
  ENTRY(g, "igk_stage_batch");
  if (count < 0 || (count > 0 && !mods)) return fail(g, IGK_EINVAL, "bad batch pointer/count");
  if (g->sharded) return fail(g, IGK_EINVAL, "igk_stage_batch: single-GPU handles only");
  if (!g->copy_stream) CK(cudaStreamCreateWithFlags(&g->copy_stream, cudaStreamNonBlocking));
  const int b = g->stage_next;
  if (g->inflight && b == g->inflight_buf) CK(cudaStreamSynchronize(g->stream));  // never under a running step
  if (count > g->sd_cap[b]) {
    CK(cudaStreamSynchronize(g->copy_stream));  // an earlier copy into this buffer has landed
    if (g->sd_mods[b]) cudaFree(g->sd_mods[b]);
    g->sd_mods[b] = nullptr;
    g->sd_cap[b] = 0;
    long long cap = grow_cap(count);
    if (cudaMalloc(&g->sd_mods[b], cap * 16) != cudaSuccess) return fail(g, IGK_ENOMEM, "batch allocation failed");
    g->sd_cap[b] = cap;
  }
  if (count > 0) {
    cudaPointerAttributes at{};
    const bool pinned = cudaPointerGetAttributes(&at, mods) == cudaSuccess && at.type == cudaMemoryTypeHost;
    cudaGetLastError();
    const void* src = mods;
    if (!pinned) {  // pageable: through the buffer's own pinned staging (the copy stays asynchronous)
      if (count > g->sh_cap[b]) {
        CK(cudaStreamSynchronize(g->copy_stream));
        if (g->sh_stage[b]) cudaFreeHost(g->sh_stage[b]);
        g->sh_stage[b] = nullptr;
        g->sh_cap[b] = 0;
        long long cap = grow_cap(count);
        CK(cudaMallocHost(&g->sh_stage[b], cap * 16));
        g->sh_cap[b] = cap;
      }
      CK(cudaEventSynchronize(g->ev_stage[b]));  // the previous copy out of this staging buffer is done
      std::memcpy(g->sh_stage[b], mods, count * 16);
      src = g->sh_stage[b];
    }
    CK(cudaMemcpyAsync(g->sd_mods[b], src, count * 16, cudaMemcpyHostToDevice, g->copy_stream));
  }
  CK(cudaEventRecord(g->ev_stage[b], g->copy_stream));
  g->sd_count[b] = count;
  g->staged = b;
  g->stage_next = b ^ 1;
  return IGK_OK;
}

igk_status igk_step_begin(igk_graph* g) {
  if (!g || g->poisoned) return IGK_ESTATE;
  ENTRY(g, "igk_step_begin");
  if (g->staged < 0 || g->inflight) return fail(g, IGK_EINVAL, "igk_step_begin: no staged batch / step in flight");
  const int b = g->staged;
  CK(cudaStreamWaitEvent(g->stream, g->ev_stage[b], 0));  // the step starts when its batch has landed
  g->inflight_buf = b;
  g->inflight_n0 = g->h_ctl->n_total;
  g->staged = -1;
  bool posted = false;
  igk_status st = step_launch(g, g->sd_mods[b], g->sd_count[b], &posted);
  if (st != IGK_OK) return st;
  g->inflight = 1;
  g->inflight_posted = posted;
  return IGK_OK;
}

igk_status igk_step_end(igk_graph* g, igk_refine_stats* stats, int64_t* first_new_id, int64_t* bad_index) {
  if (!g || g->poisoned) return IGK_ESTATE;
  ENTRY(g, "igk_step_end");
  if (!g->inflight) return fail(g, IGK_EINVAL, "igk_step_end: no step in flight");
  g->inflight = 0;
  if (bad_index) *bad_index = -1;
  if (first_new_id) *first_new_id = g->inflight_n0;
  const int b = g->inflight_buf;
  return step_complete(g, g->sd_mods[b], g->sd_count[b], g->inflight_posted, stats, bad_index);
}

igk_status igk_partition(const igk_graph* gc, int32_t* out, int64_t cap_len, int64_t* n_total) {
  igk_graph* g = const_cast<igk_graph*>(gc);
  if (!g || g->poisoned) return IGK_ESTATE;
  ENTRY(g, "igk_partition");
  long long n = g->h_ctl->n_total;
  if (n_total) *n_total = n;
  if (!out || cap_len < n) return fail(g, IGK_EINVAL, "output buffer too small");
  if (n == 0) return IGK_OK;
  k_export_part<<<592, 256, 0, g->stream>>>(g->d, n, g->d_out);
  g->launches++;
  CK(cudaGetLastError());
  CK(cudaMemcpyAsync(out, g->d_out, n * 4, cudaMemcpyDeviceToHost, g->stream));
  CK(cudaStreamSynchronize(g->stream));
  return IGK_OK;
}

igk_status igk_partition_delta(const igk_graph* gc, int32_t* pairs, int64_t cap, int64_t* count) {
  igk_graph* g = const_cast<igk_graph*>(gc);
  if (!g || g->poisoned) return IGK_ESTATE;
  ENTRY(g, "igk_partition_delta");
  if (g->delta_replaced)
    return fail(g, IGK_ESTATE, "igk_partition_delta: the partition was replaced by igk_repartition (read igk_partition)");
  const long long nd = g->h_ctl->n_delta;  // in the output head read back by the last refine / step
  if (count) *count = nd;
  if (nd == 0) return IGK_OK;
  if (!pairs || cap < nd) return fail(g, IGK_EINVAL, "delta buffer too small");
  CK(cudaMemcpyAsync(pairs, g->d.delta, nd * 8, cudaMemcpyDeviceToHost, g->stream));  // one D2H
  CK(cudaStreamSynchronize(g->stream));
  return IGK_OK;
}

igk_status igk_cut_size(const igk_graph* gc, int64_t* out) {
  igk_graph* g = const_cast<igk_graph*>(gc);
  if (!g || g->poisoned) return IGK_ESTATE;
  if (!out) return IGK_EINVAL;
  ENTRY(g, "igk_cut_size");
  if (g->sharded) {  // the global cut, all-reduced at the end of every collective call
    *out = g->cut_total;
    return IGK_OK;
  }
  CK(cudaMemcpyAsync(&g->h_ctl->cut, &g->d.ctl->cut, 8, cudaMemcpyDeviceToHost, g->stream));
  CK(cudaStreamSynchronize(g->stream));
  *out = g->h_ctl->cut;
  return IGK_OK;
}

igk_status igk_part_weights(const igk_graph* gc, int64_t* out_k) {
  igk_graph* g = const_cast<igk_graph*>(gc);
  if (!g || g->poisoned) return IGK_ESTATE;
  if (!out_k) return IGK_EINVAL;
  ENTRY(g, "igk_part_weights");
  CK(cudaMemcpyAsync(g->h_ctl->Wp, g->d.ctl->Wp, 8 * g->d.k, cudaMemcpyDeviceToHost, g->stream));
  CK(cudaStreamSynchronize(g->stream));
  for (int p = 0; p < g->d.k; p++) out_k[p] = g->h_ctl->Wp[p];
  return IGK_OK;
}

igk_status igk_num_vertices(const igk_graph* gc, int64_t* n_total, int64_t* n_active) {
  igk_graph* g = const_cast<igk_graph*>(gc);
  if (!g || g->poisoned) return IGK_ESTATE;
  ENTRY(g, "igk_num_vertices");
  if (n_total) *n_total = g->h_ctl->n_total;
  if (n_active) {  // device reduction over the labels, one 8-byte read back
    long long n = g->h_ctl->n_total;
    CK(cudaMemsetAsync(g->d_red + 258, 0, 8, g->stream));
    if (n) {
      k_count_active<<<592, 256, 0, g->stream>>>(g->d, n, g->d_red + 258);
      g->launches++;
      CK(cudaGetLastError());
    }
    long long c = 0;
    CK(cudaMemcpyAsync(&c, g->d_red + 258, 8, cudaMemcpyDeviceToHost, g->stream));
    CK(cudaStreamSynchronize(g->stream));
    *n_active = c;
  }
  return IGK_OK;
}

igk_status igk_recount(igk_graph* g, int64_t* out_cut, int64_t* out_wp) {
  if (!g || g->poisoned) return IGK_ESTATE;
  ENTRY(g, "igk_recount");
  igk_status st = launch_recount(g);
  if (st != IGK_OK) return st;
  long long red[259];
  CK(cudaMemcpyAsync(red, g->d_red, sizeof(red), cudaMemcpyDeviceToHost, g->stream));
  CK(cudaStreamSynchronize(g->stream));
  cudaEventElapsedTime(&g->ms_recount, g->ev[4], g->ev[5]);
  if (g->sharded) {  // collective: the partial cuts / entry counts of the ranks summed
    long long v[2] = {red[0], red[257]};
    st = xp_sum_host(g, v, 2);
    if (st != IGK_OK) return st;
    red[0] = v[0];
    red[257] = v[1];
  }
  g->last_entries = red[257];
  g->last_active = red[258];
  if (out_cut) *out_cut = red[0];
  if (out_wp)
    for (int p = 0; p < g->d.k; p++) out_wp[p] = red[1 + p];
  return IGK_OK;
}

igk_status igk_export_csr(const igk_graph* gc, int64_t* xadj, int64_t xadj_len, int32_t* adjncy, int32_t* adjwgt,
                          int64_t adj_len, int64_t* n_total, int64_t* n_slots) {
  igk_graph* g = const_cast<igk_graph*>(gc);
  if (!g || g->poisoned) return IGK_ESTATE;
  ENTRY(g, "igk_export_csr");
  const long long n = g->h_ctl->n_total;
  // live degree of every ID -> exclusive prefix sum (CUB) -> row gather
  // kernel: the whole CSR is built on the device and read back in three
  // copies (xadj, adjncy, adjwgt)
  long long *d_deg = nullptr, *d_off = nullptr;
  void* tmp = nullptr;
  size_t tmp_bytes = 0;
  int32_t *d_adj = nullptr, *d_w = nullptr;
  auto cleanup = [&]() {
    cudaFree(d_deg);
    cudaFree(d_off);
    cudaFree(tmp);
    cudaFree(d_adj);
    cudaFree(d_w);
  };
  const long long nn = std::max<long long>(n, 1);
  if (cudaMalloc(&d_deg, (nn + 1) * 8) != cudaSuccess || cudaMalloc(&d_off, (nn + 1) * 8) != cudaSuccess) {
    cleanup();
    return fail(g, IGK_ENOMEM, "export: allocation failed");
  }
  cudaMemsetAsync(d_deg, 0, (nn + 1) * 8, g->stream);
  if (n) k_export_deg<<<592, 256, 0, g->stream>>>(g->d, n, d_deg);
  cub::DeviceScan::ExclusiveSum(nullptr, tmp_bytes, d_deg, d_off, n + 1, g->stream);
  if (cudaMalloc(&tmp, std::max<size_t>(tmp_bytes, 1)) != cudaSuccess) {
    cleanup();
    return fail(g, IGK_ENOMEM, "export: allocation failed");
  }
  cub::DeviceScan::ExclusiveSum(tmp, tmp_bytes, d_deg, d_off, n + 1, g->stream);
  g->launches += n ? 2 : 1;
  long long tot = 0;
  if (cudaMemcpyAsync(&tot, d_off + n, 8, cudaMemcpyDeviceToHost, g->stream) != cudaSuccess ||
      cudaStreamSynchronize(g->stream) != cudaSuccess) {
    cleanup();
    CK(cudaGetLastError());
    return fail(g, IGK_ECUDA, "export failed");
  }
  if (n_total) *n_total = n;
  if (n_slots) *n_slots = tot;
  if (!xadj) {
    cleanup();
    return IGK_OK;
  }
  if (xadj_len < n + 1 || adj_len < tot || !adjncy) {
    cleanup();
    return fail(g, IGK_EINVAL, "export buffers too small");
  }
  if (cudaMalloc(&d_adj, std::max<long long>(tot, 1) * 4) != cudaSuccess ||
      cudaMalloc(&d_w, std::max<long long>(tot, 1) * 4) != cudaSuccess) {
    cleanup();
    return fail(g, IGK_ENOMEM, "export: allocation failed");
  }
  if (n) {
    k_export_rows<<<1184, 256, 0, g->stream>>>(g->d, n, d_off, d_adj, d_w);
    g->launches++;
  }
  cudaError_t e = cudaGetLastError();
  if (e == cudaSuccess) e = cudaMemcpyAsync(xadj, d_off, (n + 1) * 8, cudaMemcpyDeviceToHost, g->stream);
  if (e == cudaSuccess && tot) e = cudaMemcpyAsync(adjncy, d_adj, tot * 4, cudaMemcpyDeviceToHost, g->stream);
  if (e == cudaSuccess && tot && adjwgt) e = cudaMemcpyAsync(adjwgt, d_w, tot * 4, cudaMemcpyDeviceToHost, g->stream);
  if (e == cudaSuccess) e = cudaStreamSynchronize(g->stream);
  cleanup();
  CK(e);
  return IGK_OK;
}

igk_status igk_debug_set_profile(igk_graph* g, int32_t on) {
  if (!g || g->poisoned) return IGK_ESTATE;
  g->prof = on != 0;
  g->debug_phases = on != 0 || getenv("IGK_DEBUG_PHASES") != nullptr || getenv("IGK_DEBUG_ARRIVALS") != nullptr;
  return IGK_OK;
}

int32_t igk_debug_phase_work(const igk_graph* gc, int64_t* scanned, int64_t* items, int32_t cap) {
  igk_graph* g = const_cast<igk_graph*>(gc);
  if (!g || g->poisoned) return 0;
  ENTRY(g, "igk_debug_phase_work");
  long long buf[16];
  if (cudaMemcpyAsync(buf, &g->d.ctl->phscan[0], sizeof(buf), cudaMemcpyDeviceToHost, g->stream) != cudaSuccess ||
      cudaStreamSynchronize(g->stream) != cudaSuccess)
    return 0;
  const int n = std::min<int>(cap, PH_N);
  for (int i = 0; i < n; i++) {
    if (scanned) scanned[i] = buf[i];
    if (items) items[i] = buf[8 + i];
  }
  return n;
}

igk_status igk_nccl_unique_id(void* out, int64_t len) {
  if (!out || len < (int64_t)sizeof(ncclUniqueId)) return IGK_EINVAL;
  const NcclApi* api = nccl_api();
  if (!api) return IGK_ENCCL;
  ncclUniqueId id;
  if (api->get_unique_id(&id) != ncclSuccess) return IGK_ENCCL;
  std::memcpy(out, &id, sizeof id);
  return IGK_OK;
}

int32_t igk_debug_paths(const igk_graph* gc, int64_t* out, int32_t cap) {
  igk_graph* g = const_cast<igk_graph*>(gc);
  if (!g || g->poisoned || !out) return 0;
  ENTRY(g, "igk_debug_paths");
  long long dev[PA_N_DEV];
  if (cudaMemcpyAsync(dev, g->d.ctl->paths, sizeof(dev), cudaMemcpyDeviceToHost, g->stream) != cudaSuccess ||
      cudaStreamSynchronize(g->stream) != cudaSuccess)
    return 0;
  const long long host[] = {g->compactions, g->n_grow, g->n_split, g->n_fused, g->n_notice_fallback};
  int32_t n = 0;
  for (int i = 0; i < PA_N_DEV && n < cap; i++) out[n++] = dev[i];
  for (long long h : host)
    if (n < cap) out[n++] = h;
  return n;
}

int64_t igk_kernel_launches(const igk_graph* g) { return g ? g->launches : 0; }

igk_status igk_compact(igk_graph* g) {
  if (!g || g->poisoned) return IGK_ESTATE;
  ENTRY(g, "igk_compact");
  igk_status st = sync_ctl(g, -1);
  if (st != IGK_OK) return st;
  return compact_slab(g, 0);
}

igk_status igk_store_stats(const igk_graph* g, int64_t* n_total, int64_t* n_active, int64_t* adj_entries,
                           int64_t* slab_top, int64_t* slab_cap) {
  if (!g || g->poisoned) return IGK_ESTATE;
  if (n_total) *n_total = g->h_ctl->n_total;
  if (n_active) *n_active = g->last_active;
  if (adj_entries) *adj_entries = g->last_entries;
  if (slab_top) *slab_top = g->h_ctl->slab_top;
  if (slab_cap) *slab_cap = g->d.slot_cap;
  return IGK_OK;
}

igk_status igk_last_kernel_ms(const igk_graph* g, float* refine_ms, float* apply_ms, float* recount_ms) {
  if (!g) return IGK_ESTATE;
  DevGuard dev_guard(g->device);
  if (g->ms_pending) {  // fast path: the step returned before its end event completed
    igk_graph* gm = const_cast<igk_graph*>(g);
    cudaEventSynchronize(gm->ev[1]);
    cudaEventElapsedTime(&gm->ms_refine, gm->ev[0], gm->ev[1]);
    gm->ms_pending = 0;
  }
  if (refine_ms) *refine_ms = g->ms_refine;
  if (apply_ms) *apply_ms = g->ms_apply;
  if (recount_ms) *recount_ms = g->ms_recount;
  return IGK_OK;
}

int32_t igk_debug_arrivals(const igk_graph* g, int32_t which, int64_t* out, int32_t cap) {
  if (!g || !g->d.dbg || !out) return 0;
  if (which == 2) {  // per-warp diagnostics of the last F1 commit pass: 4096 times, then 4096 values
    std::vector<unsigned long long> h(16384);
    if (cudaMemcpy(h.data(), g->d.dbg + kDbgWarp, h.size() * 8, cudaMemcpyDeviceToHost) != cudaSuccess) return 0;
    for (size_t i = 0; i < h.size() && (int64_t)i < cap; i++) out[i] = (int64_t)h[i];
    return g->grid_refine_k * (kThreads / 32);
  }
  int grid = which == 0 ? g->grid_apply : g->grid_refine_k;
  std::vector<unsigned long long> h((size_t)128 * grid);
  if (cudaMemcpy(h.data(), g->d.dbg, h.size() * 8, cudaMemcpyDeviceToHost) != cudaSuccess) return 0;
  for (size_t i = 0; i < h.size() && (int64_t)i < cap; i++) out[i] = (int64_t)h[i];
  return grid;
}

int32_t igk_debug_phase_times(const igk_graph* g, int32_t which, int32_t* ids, int64_t* t_ns, int32_t cap) {
  if (!g || which < 0 || which > 1) return 0;
  const auto& v = g->ph[which];
  int32_t n = (int32_t)std::min<size_t>(v.size(), (size_t)std::max(cap, 0));
  for (int32_t i = 0; i < n; i++) {
    if (ids) ids[i] = v[i].first;
    if (t_ns) t_ns[i] = (int64_t)(v[i].second - v[0].second);
  }
  return n;
}

const char* igk_last_error(const igk_graph* g) {
  return g ? g->err.c_str() : (t_create_err.empty() ? "null handle" : t_create_err.c_str());
}

void igk_destroy(igk_graph* g) {
  if (!g) return;
  DevGuard dev_guard(g->device);
  cudaStreamSynchronize(g->stream);
  if (g->p2p) {
    p2p_teardown(g);
    if (g->p2p_mem) cudaFree(g->p2p_mem);
    if (g->p2p_bar) cudaFree(g->p2p_bar);
  }
  if (g->nccl && nccl_api()) nccl_api()->destroy((ncclComm_t)g->nccl);
  if (g->xp_host) cudaFreeHost(g->xp_host);
  if (g->sort_tmp) cudaFree(g->sort_tmp);
  for (void* p : g->allocs) cudaFree(p);
  if (g->d.hkeys) cudaFree(g->d.hkeys);
  if (g->d.hcnt) cudaFree(g->d.hcnt);
  if (g->d.newid) cudaFree(g->d.newid);
  if (g->d_mods) cudaFree(g->d_mods);
  if (g->h_stage) cudaFreeHost(g->h_stage);
  if (g->h_ctl) cudaFreeHost(g->h_ctl);
  if (g->h_map) cudaFreeHost(g->h_map);
  if (g->h_flag) cudaFreeHost(g->h_flag);
  for (auto& e : g->ev)
    if (e) cudaEventDestroy(e);
  for (int b = 0; b < 2; b++) {
    if (g->ev_stage[b]) cudaEventDestroy(g->ev_stage[b]);
    if (g->sd_mods[b]) cudaFree(g->sd_mods[b]);
    if (g->sh_stage[b]) cudaFreeHost(g->sh_stage[b]);
  }
  if (g->copy_stream) cudaStreamDestroy(g->copy_stream);
  delete g;
}

}  // extern "C"
