// fgp.cuh -- NEXT-2: the GPU kernels of IGK-FGP v1, the full partitioner
// (G-kway with the paper's constrained coarsening, Sec. IV; group
// size s and the stop rules of P:273), readings F1-F6 of DESIGN.md 4.
//
// Per coarsening level (igk.cu igk_fgp_partition drives them, with CUB sorts / scans
// in between):
//   k_fgp_select   heaviest incident edge per vertex, warp per vertex; for a
//                  fixed vertex the global edge order (w desc, min ID, max ID)
//                  reduces to (w desc, neighbour ID asc): one 64-bit key
//   k_fgp_roots    self-pointers and the smaller vertex of each mutual pair
//   k_fgp_jump     one synchronous pointer-jumping iteration + join labels
//   k_fgp_keys     (subset root, label) sort keys for the stable radix sort
//   k_fgp_groups   group starts in the sorted order (subset start, or every
//                  s-th vertex of a subset), singleton count
//   k_fgp_cmap     vertex -> group (coarse vertex) from the scanned starts
//   k_fgp_cvw      coarse vertex weights
//   k_fgp_edges    inter-group entries as (coarse u, coarse x) keys + weight
//   k_fgp_rows     coarse CSR rows from the reduced, sorted keys
//   k_fgp_initial  greedy graph growing on the coarsest graph (one thread:
//                  a few thousand vertices)
//   k_fgp_project  fine part = part of the vertex's group
// and per finer level the label-propagation passes of reading F7:
//   k_lp_gain      warp per vertex: per-part connectivity in shared memory,
//                  best other part (conn desc, part asc), gain
//   k_lp_filter    a candidate survives iff it beats every candidate
//                  neighbour in (gain desc, ID asc)
//   k_lp_keys / k_lp_segs / k_lp_admit   (target, gain desc, ID asc) order
//                  by a stable radix sort of the survivors (listed in ID
//                  order), running weight per target, admitted while
//                  W_b + running weight <= cap
#pragma once
#include "common.cuh"

namespace igk {

__global__ void k_fgp_select(long long n, const int64_t* xadj, const int32_t* adj, const int32_t* w, int32_t* sel) {
  const long long gw = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const long long nw = ((long long)gridDim.x * blockDim.x) >> 5;
  const int lane = threadIdx.x & 31;
  for (long long v = gw; v < n; v += nw) {
    unsigned long long best = 0;  // key = w << 32 | (~x): max wins; 0 = none
    for (long long j = xadj[v] + lane; j < xadj[v + 1]; j += 32) {
      const unsigned long long key = ((unsigned long long)(unsigned)w[j] << 32) | (0xffffffffu - (unsigned)adj[j]);
      best = key > best ? key : best;
    }
#pragma unroll
    for (int o = 16; o; o >>= 1) {
      const unsigned long long b = __shfl_xor_sync(0xffffffffu, best, o);
      best = b > best ? b : best;
    }
    if (lane == 0) sel[v] = best ? (int32_t)(0xffffffffu - (unsigned)(best & 0xffffffffu)) : (int32_t)v;
  }
}

// the smallest isolated vertex (it selected itself): every isolated vertex
// points at it (reading F1), so they merge in groups like any other subset
__global__ void k_fgp_iso(long long n, const int32_t* sel, int* iso0) {
  for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (long long)gridDim.x * blockDim.x)
    if (sel[v] == v) atomicMin(iso0, (int)v);
}
__global__ void k_fgp_roots(long long n, int32_t* sel, const int* iso0p, int32_t* P, int32_t* label, int* left) {
  const int iso0 = *iso0p;
  int c = 0;
  for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (long long)gridDim.x * blockDim.x) {
    int32_t s = sel[v];
    if (s == v) s = iso0;  // isolated (a vertex with an edge never selects itself)
    const bool root = s == v || (sel[s] == v && v < s);
    P[v] = root ? (int32_t)v : s;
    label[v] = root ? 0 : -1;
    c += !root;
  }
  c = warp_sum(c);
  if ((threadIdx.x & 31) == 0 && c) atomicAdd(left, c);
}

// iteration t: label the vertices whose pointer is a root (read at the start
// of the iteration), then P' = P o P -- both from P_in (synchronous)
__global__ void k_fgp_jump(long long n, const int32_t* Pin, int32_t* Pout, int32_t* label, int t, int* left) {
  int c = 0;
  for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (long long)gridDim.x * blockDim.x) {
    const int32_t p = Pin[v];
    const int32_t pp = Pin[p];
    if (label[v] < 0) {
      if (pp == p) label[v] = t;
      else c++;
    }
    Pout[v] = pp;
  }
  c = warp_sum(c);
  if ((threadIdx.x & 31) == 0 && c) atomicAdd(left, c);
}

__global__ void k_fgp_keys(long long n, const int32_t* P, const int32_t* label, unsigned long long* key,
                           int32_t* val) {
  for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (long long)gridDim.x * blockDim.x) {
    key[v] = ((unsigned long long)(unsigned)P[v] << 8) | (unsigned)label[v];
    val[v] = (int32_t)v;
  }
}

// segment (subset) starts; segstart[i] = the index of i's subset start,
// filled by a max-scan of these marks
__global__ void k_fgp_segmark(long long n, const unsigned long long* skey, long long* mark) {
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x)
    mark[i] = (i == 0 || (skey[i] >> 8) != (skey[i - 1] >> 8)) ? i : 0;
}
__global__ void k_fgp_groups(long long n, const long long* segstart, int s, int32_t* flag) {
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x)
    flag[i] = ((i - segstart[i]) % s) == 0;
}
// vertex -> group (gid = inclusive scan of the starts, minus one); singletons
// counted (a group start followed by a start or the end)
__global__ void k_fgp_cmap(long long n, const int32_t* flag, const int32_t* gid, const int32_t* sval, int32_t* cmap,
                           int* singles) {
  int c = 0;
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
    cmap[sval[i]] = gid[i] - 1;
    c += flag[i] && (i + 1 == n || flag[i + 1]);
  }
  c = warp_sum(c);
  if ((threadIdx.x & 31) == 0 && c) atomicAdd(singles, c);
}

__global__ void k_fgp_cvw(long long n, const int32_t* cmap, const int32_t* vw, int32_t* cvw) {
  for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (long long)gridDim.x * blockDim.x)
    atomicAdd(cvw + cmap[v], vw[v]);
}

// inter-group entries (a, b, w) with a != b; order irrelevant (sorted next)
__global__ void k_fgp_edges(long long n, const int64_t* xadj, const int32_t* adj, const int32_t* w,
                            const int32_t* cmap, unsigned long long* ekey, int32_t* ew, unsigned long long* cnt) {
  const long long gw = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const long long nw = ((long long)gridDim.x * blockDim.x) >> 5;
  const int lane = threadIdx.x & 31;
  for (long long v = gw; v < n; v += nw) {
    const unsigned a = (unsigned)cmap[v];
    for (long long j0 = xadj[v]; j0 < xadj[v + 1]; j0 += 32) {
      const long long j = j0 + lane;
      unsigned b = a;
      if (j < xadj[v + 1]) b = (unsigned)cmap[adj[j]];
      const bool keep = j < xadj[v + 1] && b != a;
      const unsigned m = __ballot_sync(0xffffffffu, keep);
      unsigned long long base = 0;
      if (lane == 0 && m) base = atomicAdd(cnt, (unsigned long long)__popc(m));
      base = __shfl_sync(0xffffffffu, base, 0);
      if (keep) {
        const unsigned long long pos = base + __popc(m & ((1u << lane) - 1u));
        ekey[pos] = ((unsigned long long)a << 32) | b;
        ew[pos] = w[j];
      }
    }
  }
}

__global__ void k_fgp_rowcount(long long nu, const unsigned long long* ukey, int64_t* cnt) {
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < nu; i += (long long)gridDim.x * blockDim.x)
    atomicAdd((unsigned long long*)(cnt + (ukey[i] >> 32)), 1ull);
}
__global__ void k_fgp_rows(long long nu, const unsigned long long* ukey, int32_t* cadj) {
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < nu; i += (long long)gridDim.x * blockDim.x)
    cadj[i] = (int32_t)(ukey[i] & 0xffffffffu);
}

// greedy graph growing (reading F5): BFS from the smallest unvisited ID,
// neighbours in row order (rows are sorted), the part advances once the
// running weight reaches (p + 1) W / k
__global__ void k_fgp_initial(long long n, const int64_t* xadj, const int32_t* adj, const int32_t* vw, int k,
                              int32_t* part, uint8_t* vis, int32_t* queue) {
  if (blockIdx.x != 0 || threadIdx.x != 0) return;
  long long W = 0;
  for (long long v = 0; v < n; v++) {
    W += vw[v];
    vis[v] = 0;
  }
  long long acc = 0;
  int p = 0;
  for (long long s = 0; s < n; s++) {
    if (vis[s]) continue;
    long long qh = 0, qt = 0;
    queue[qt++] = (int32_t)s;
    vis[s] = 1;
    while (qh < qt) {
      const int32_t v = queue[qh++];
      part[v] = p;
      acc += vw[v];
      if (p < k - 1 && acc * k >= (long long)(p + 1) * W) p++;
      for (long long j = xadj[v]; j < xadj[v + 1]; j++) {
        const int32_t x = adj[j];
        if (!vis[x]) {
          vis[x] = 1;
          queue[qt++] = x;
        }
      }
    }
  }
}

__global__ void k_fgp_project(long long n, const int32_t* cmap, const int32_t* cpart, int32_t* part) {
  for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (long long)gridDim.x * blockDim.x)
    part[v] = cpart[cmap[v]];
}

// ---- F7 label propagation --------------------------------------------------
constexpr int kLpThreads = 256;
__global__ void k_lp_pw(long long n, const int32_t* part, const int32_t* vw, unsigned long long* W) {
  for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (long long)gridDim.x * blockDim.x)
    atomicAdd(W + part[v], (unsigned long long)vw[v]);
}

__global__ void __launch_bounds__(kLpThreads) k_lp_gain(long long n, const int64_t* xadj, const int32_t* adj,
                                                        const int32_t* w, const int32_t* part, int k, int32_t* tgt,
                                                        int32_t* gain) {
  __shared__ int conn_s[kLpThreads / 32][kMaxK + 2];
  const int lane = threadIdx.x & 31, wi = threadIdx.x >> 5;
  int* conn = conn_s[wi];
  for (int p = lane; p < k; p += 32) conn[p] = 0;
  __syncwarp();
  const long long nw = ((long long)gridDim.x * blockDim.x) >> 5;
  for (long long v = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5; v < n; v += nw) {
    const long long b0 = xadj[v], b1 = xadj[v + 1];
    for (long long j = b0 + lane; j < b1; j += 32) atomicAdd(conn + part[adj[j]], w[j]);
    __syncwarp();
    const int a = part[v];
    unsigned long long best = 0;  // (conn << 8) | (255 - p): max = (conn desc, p asc)
    for (int p = lane; p < k; p += 32) {
      const unsigned long long key = ((unsigned long long)(unsigned)conn[p] << 8) | (unsigned)(255 - p);
      if (p != a && key > best) best = key;
    }
#pragma unroll
    for (int o = 16; o; o >>= 1) {
      const unsigned long long x = __shfl_xor_sync(0xffffffffu, best, o);
      best = x > best ? x : best;
    }
    const long long cb = (long long)(best >> 8), ca = conn[a];
    __syncwarp();
    for (int p = lane; p < k; p += 32) conn[p] = 0;
    __syncwarp();
    if (lane == 0) {
      const bool cand = cb - ca > 0;
      tgt[v] = cand ? 255 - (int)(best & 0xff) : -1;
      gain[v] = cand ? (int32_t)(cb - ca) : 0;
    }
  }
}

__global__ void k_lp_filter(long long n, const int64_t* xadj, const int32_t* adj, const int32_t* tgt,
                            const int32_t* gain, int32_t* flag) {
  const int lane = threadIdx.x & 31;
  const long long nw = ((long long)gridDim.x * blockDim.x) >> 5;
  for (long long v = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5; v < n; v += nw) {
    if (tgt[v] < 0) {
      if (lane == 0) flag[v] = 0;
      continue;
    }
    const int32_t gv = gain[v];
    bool beaten = false;
    for (long long j = xadj[v] + lane; j < xadj[v + 1] && !beaten; j += 32) {
      const int32_t u = adj[j];
      if (tgt[u] >= 0) {
        const int32_t gu = gain[u];
        beaten = gu > gv || (gu == gv && u < v);
      }
    }
    beaten = __any_sync(0xffffffffu, beaten);
    if (lane == 0) flag[v] = !beaten;
  }
}

__global__ void k_lp_iota(long long n, int32_t* ids) {
  for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (long long)gridDim.x * blockDim.x)
    ids[v] = (int32_t)v;
}

// key = target << 31 | (INT32_MAX - gain): ascending = (target, gain desc)
__global__ void k_lp_keys(const int* nm, const int32_t* sel, const int32_t* tgt, const int32_t* gain,
                          unsigned long long* key) {
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < *nm; i += (long long)gridDim.x * blockDim.x) {
    const int32_t v = sel[i];
    key[i] = ((unsigned long long)tgt[v] << 31) | (unsigned)(0x7fffffff - gain[v]);
  }
}

__global__ void k_lp_segs(const int* nm, const unsigned long long* skey, const int32_t* sid, const int32_t* vw,
                          long long* wts, long long* mark) {
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < *nm; i += (long long)gridDim.x * blockDim.x) {
    wts[i] = vw[sid[i]];
    mark[i] = (i == 0 || (skey[i] >> 31) != (skey[i - 1] >> 31)) ? i : 0;
  }
}

// admission against the snapshot W; part and the weight deltas written here,
// W itself updated by k_lp_applyw after the launch
__global__ void k_lp_admit(const int* nm, const unsigned long long* skey, const int32_t* sid, const long long* incl,
                           const long long* segstart, const unsigned long long* W, long long cap, const int32_t* vw,
                           const int32_t* gain, int32_t* part, long long* dW, unsigned long long* cnt) {
  unsigned long long moved = 0, red = 0;
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < *nm; i += (long long)gridDim.x * blockDim.x) {
    const int b = (int)(skey[i] >> 31);
    const long long s0 = segstart[i];
    const long long run = incl[i] - (s0 > 0 ? incl[s0 - 1] : 0);
    if ((long long)W[b] + run <= cap) {
      const int32_t v = sid[i];
      const int a = part[v];
      atomicAdd((unsigned long long*)(dW + a), (unsigned long long)(-(long long)vw[v]));
      atomicAdd((unsigned long long*)(dW + b), (unsigned long long)vw[v]);
      part[v] = b;
      moved++;
      red += (unsigned long long)gain[v];
    }
  }
  if (moved) {
    atomicAdd(cnt, moved);
    atomicAdd(cnt + 1, red);
  }
}

__global__ void k_lp_applyw(int k, unsigned long long* W, long long* dW) {
  for (int p = threadIdx.x; p < k; p += blockDim.x) {
    W[p] += (unsigned long long)dW[p];
    dW[p] = 0;
  }
}

}  // namespace igk
