// common.cuh -- device state, constants and warp/block helpers for libigk.
//
// Product code (sm_100a).  Shares nothing with oracle/ (see DESIGN.md 5).
#pragma once
#include <cooperative_groups.h>
#include <cuda_runtime.h>
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
constexpr int kThreads = 512;       // persistent-kernel block size
constexpr int kWarps = kThreads / 32;
constexpr int kThreadDeg = 32;      // degree <= this: one thread per vertex; above: one warp
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

struct Ctl {
  long long n_total;   // vertex IDs in use
  long long slab_top;  // bump pointer of the adjacency slab
  long long W;         // total active vertex weight
  long long cut;       // maintained cut (placed endpoints only)
  long long Wp[256];   // part weights
  long long tot3[3][256];  // per round (mod 3): weight of selected moves per target part
  long long st_out[ST_N];  // stats of the last refine (copied at its end)
  long long slab_top0;     // slab_top before the current apply (rollback)
  long long err_idx;   // lowest invalid modifier index (kNoErr = none)
  long long st[ST_N];  // refine stats
  int err_nomem;
  int n_ins;
  int nA;              // affected list length
  int npsi[2];         // pseudo list lengths (double buffer)
  int ncand;           // candidate list length
  int nN;              // expansion list length
  int ngrow;           // relocation list length
  int ndirty;          // compaction list length
  int nr3;             // restoration candidate list length
  int applied3[3];     // moves applied per round (mod 3)
  int selected3[3];    // moves selected per round (mod 3)
};

// ---------------------------------------------------------------------------
// all device pointers of one handle, passed by value to every kernel
// ---------------------------------------------------------------------------
struct Dev {
  int32_t k;
  int64_t n_cap;     // vertex capacity
  int64_t slot_cap;  // slab capacity (entries)
  int32_t slack_min;
  int32_t idbits;    // bits to hold any vertex ID < n_cap
  // graph store (S0)
  int64_t* off;      // slab offset of each vertex's dense prefix
  int32_t* deg;      // prefix length
  int32_t* capv;     // capacity
  int32_t* adj;      // neighbour IDs
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
  int32_t* psi[2];
  int32_t* cand;
  int32_t* Nlist;
  int32_t* glist;    // grow / relocation list
  int32_t* dlist;    // dirty list
  int2* r3list;      // (vertex, loss) restoration candidates
  int64_t* reloc;    // new slab offset for relocated vertices
  // per-vertex move results (rounds)
  uint8_t* tgt;
  int32_t* gain;
  int32_t* pw;
  uint32_t* meta;    // per psi index: bit31 selected | d0 << 8 | p*
  // selection histograms
  long long* hist0;  // [256][256] digit-0 weights per part
  long long* histR;  // [3][256][256] pass histograms
  // apply scratch
  unsigned long long* hkeys;  // dup-detection hash (keys)
  int32_t* hcnt;              // dup-detection hash (counts)
  int64_t hmask;
  int32_t* blkcnt;            // per-block counts for chunked scans
  int32_t* newid;             // per modifier: new vertex ID of a VERTEX_INSERT
  Ctl* ctl;
};

// ---------------------------------------------------------------------------
// helpers
// ---------------------------------------------------------------------------
__device__ __forceinline__ long long ldv(const long long* p) { return *(volatile const long long*)p; }
__device__ __forceinline__ int ldv(const int* p) { return *(volatile const int*)p; }
__device__ __forceinline__ uint8_t ld_part(const uint8_t* p, int64_t i) { return __ldcg(p + i); }

__device__ __forceinline__ int lane_id() { return threadIdx.x & 31; }
__device__ __forceinline__ int warp_id() { return threadIdx.x >> 5; }

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

__device__ __forceinline__ int edge_w(const int32_t* adjw, int64_t j) { return adjw ? __ldg(adjw + j) : 1; }
__device__ __forceinline__ int vert_w(const int32_t* vw, int64_t v) { return vw ? __ldg(vw + v) : 1; }

// cap(W) = max(floor(W (1e6 + e) / (1e6 k)), ceil(W / k))  (reading Q4)
__host__ __device__ __forceinline__ long long cap_of(long long W, long long e_ppm, int k) {
  unsigned __int128 num = (unsigned __int128)(unsigned long long)W * (unsigned long long)(1000000 + e_ppm);
  unsigned long long den = 1000000ull * (unsigned long long)k;
  long long a = (long long)(num / den);
  long long b = (W + k - 1) / k;
  return a > b ? a : b;
}

}  // namespace igk
