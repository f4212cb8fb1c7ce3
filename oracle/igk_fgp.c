/*
 * igk_fgp.c -- CPU oracle of IGK-FGP v1, the full partitioner of SURVEY 8(f)
 * NEXT-2 (G-kway with the paper's constrained coarsening, Sec. IV).
 *
 * TEST INFRASTRUCTURE ONLY (see igk_oracle.h): nothing in the product path
 * includes, links or calls this file.
 *
 * The paper describes the method in prose only (Fig. 3) and fixes
 * the parameters at P:273 (group size s = 6; coarsening stops when fewer
 * than 35 k vertices remain or fewer than 90% of the vertices could be
 * coarsened).  Everything it leaves open is a reading (F1-F7):
 *
 *  per level l, on G_l (vertex weights, edge weights):
 *   1. selection (F1): every vertex points at the neighbour across its
 *      heaviest incident edge, edges totally ordered by (w desc, min ID asc,
 *      max ID asc); an isolated vertex points at the smallest isolated
 *      vertex (that one at itself), so isolated vertices form one subset and
 *      merge in groups like any other (merging them cuts no edge).  In that
 *      order the pointer graph's only cycles are mutual pairs.
 *   2. union-find with join labels (F2; "labeling each vertex with the
 *      iteration in which it joins a subset"): roots = self-pointers
 *      and the smaller vertex of each mutual pair; synchronous pointer
 *      jumping P <- P o P; label(v) = the first iteration t >= 1 at whose
 *      start P(v) is a root (roots: 0); subset(v) = the final P(v).
 *   3. constrained grouping (F3; "sort the vertices based on their
 *      labels and divide them into groups"): inside each subset, vertices
 *      sorted by (label, ID); consecutive runs of s vertices form groups;
 *      groups numbered in (subset root, run index) order = coarse IDs.
 *   4. stop rules (F4): if the vertices in groups of size >= 2 are
 *      fewer than 90% of n_l, G_l is the coarsest graph; otherwise contract
 *      (weights summed, edges inside a group dropped, parallel edges summed,
 *      rows sorted by ID) and stop once n_{l+1} < 35 k (or no progress, or
 *      32 levels).
 *  initial partition (F5; the paper defers to G-kway): greedy graph growing
 *      on the coarsest graph -- BFS from the smallest unvisited ID,
 *      neighbours in ID order, the current part advances once the running
 *      weight reaches (p + 1) W / k.
 *  coarsest refinement (F6): the initial partition is refined with the
 *      global boundary refinement of NEXT-1 (ora_refine_global: R1-R4, incl.
 *      R3 restoration of any overweight part), repeated while a pass lowers
 *      the cut (at most 8 passes).
 *  uncoarsening (F7): at every finer level the partition is projected (each
 *      vertex takes its group's part) and refined by synchronous
 *      label-propagation passes (fgp_lp_pass below), until a pass moves
 *      nothing (at most 16 passes).
 */
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include "igk_oracle.h"

typedef struct {
  int64_t n;
  int64_t* xadj;
  int32_t* adj;
  int32_t* w;
  int32_t* vw;
} fcsr;

static void* fxalloc(size_t n, size_t s) {
  void* p = calloc(n ? n : 1, s);
  if (!p) {
    fprintf(stderr, "oracle fgp: out of memory\n");
    abort();
  }
  return p;
}
static void fcsr_free(fcsr* G) {
  free(G->xadj);
  free(G->adj);
  free(G->w);
  free(G->vw);
  memset(G, 0, sizeof *G);
}

/* 1. heaviest incident edge, edges ordered by (w desc, min asc, max asc) */
static void fgp_select(const fcsr* G, int32_t* sel) {
  for (int64_t v = 0; v < G->n; v++) {
    int64_t best = v, bw = -1, blo = 0, bhi = 0;
    for (int64_t j = G->xadj[v]; j < G->xadj[v + 1]; j++) {
      const int64_t x = G->adj[j], ww = G->w[j];
      const int64_t lo = v < x ? v : x, hi = v < x ? x : v;
      if (ww > bw || (ww == bw && (lo < blo || (lo == blo && hi < bhi)))) {
        best = x;
        bw = ww;
        blo = lo;
        bhi = hi;
      }
    }
    sel[v] = (int32_t)best;
  }
  int64_t iso0 = -1; /* the smallest isolated vertex */
  for (int64_t v = 0; v < G->n; v++)
    if (G->xadj[v] == G->xadj[v + 1]) {
      if (iso0 < 0) iso0 = v;
      sel[v] = (int32_t)iso0;
    }
}

/* 2. roots, synchronous pointer jumping, join labels */
static void fgp_union(const fcsr* G, const int32_t* sel, int32_t* root, int32_t* label) {
  const int64_t n = G->n;
  int32_t* P = (int32_t*)fxalloc(n, sizeof(int32_t));
  int32_t* Q = (int32_t*)fxalloc(n, sizeof(int32_t));
  for (int64_t v = 0; v < n; v++) {
    const int32_t s = sel[v];
    const int is_root = s == v || (sel[s] == v && v < s);
    P[v] = is_root ? (int32_t)v : s;
    label[v] = is_root ? 0 : -1;
  }
  int left = 0;
  for (int64_t v = 0; v < n; v++) left += label[v] < 0;
  for (int t = 1; left > 0; t++) {
    for (int64_t v = 0; v < n; v++)
      if (label[v] < 0 && P[P[v]] == P[v]) {
        label[v] = t;
        left--;
      }
    for (int64_t v = 0; v < n; v++) Q[v] = P[P[v]];
    int32_t* T = P;
    P = Q;
    Q = T;
  }
  for (int64_t v = 0; v < n; v++) root[v] = P[v];
  free(P);
  free(Q);
}

typedef struct {
  int32_t root, label, id;
} fgkey;
static int cmp_fgkey(const void* a, const void* b) {
  const fgkey* x = (const fgkey*)a;
  const fgkey* y = (const fgkey*)b;
  if (x->root != y->root) return x->root < y->root ? -1 : 1;
  if (x->label != y->label) return x->label < y->label ? -1 : 1;
  return x->id < y->id ? -1 : (x->id > y->id);
}

/* 3. groups of s in (root, label, ID) order; returns the number of groups,
 * cmap[v] = group of v, *coarsenable = vertices in groups of size >= 2 */
static int64_t fgp_group(const fcsr* G, const int32_t* root, const int32_t* label, int32_t s, int32_t* cmap,
                         int64_t* coarsenable) {
  const int64_t n = G->n;
  fgkey* ks = (fgkey*)fxalloc(n, sizeof(fgkey));
  for (int64_t v = 0; v < n; v++) {
    ks[v].root = root[v];
    ks[v].label = label[v];
    ks[v].id = (int32_t)v;
  }
  qsort(ks, n, sizeof(fgkey), cmp_fgkey);
  int64_t ng = 0, co = 0;
  for (int64_t i = 0; i < n;) {
    int64_t e = i;
    while (e < n && ks[e].root == ks[i].root) e++;  /* one subset: [i, e) */
    for (int64_t a = i; a < e; a += s) {
      const int64_t b = a + s < e ? a + s : e;
      for (int64_t t = a; t < b; t++) cmap[ks[t].id] = (int32_t)ng;
      if (b - a >= 2) co += b - a;
      ng++;
    }
    i = e;
  }
  free(ks);
  *coarsenable = co;
  return ng;
}

typedef struct {
  int32_t a, b;
  int64_t w;
} fedge;
static int cmp_fedge(const void* x, const void* y) {
  const fedge* p = (const fedge*)x;
  const fedge* q = (const fedge*)y;
  if (p->a != q->a) return p->a < q->a ? -1 : 1;
  return p->b < q->b ? -1 : (p->b > q->b);
}

/* contraction: summed vertex weights, inter-group edges summed, rows sorted */
static void fgp_contract(const fcsr* G, const int32_t* cmap, int64_t nc, fcsr* C) {
  C->n = nc;
  C->vw = (int32_t*)fxalloc(nc, sizeof(int32_t));
  for (int64_t v = 0; v < G->n; v++) C->vw[cmap[v]] += G->vw[v];
  const int64_t m2 = G->xadj[G->n];
  fedge* es = (fedge*)fxalloc(m2, sizeof(fedge));
  int64_t ne = 0;
  for (int64_t v = 0; v < G->n; v++)
    for (int64_t j = G->xadj[v]; j < G->xadj[v + 1]; j++) {
      const int32_t a = cmap[v], b = cmap[G->adj[j]];
      if (a == b) continue;
      es[ne].a = a;
      es[ne].b = b;
      es[ne].w = G->w[j];
      ne++;
    }
  qsort(es, ne, sizeof(fedge), cmp_fedge);
  int64_t u = 0;
  for (int64_t i = 0; i < ne; i++) {
    if (u > 0 && es[u - 1].a == es[i].a && es[u - 1].b == es[i].b) es[u - 1].w += es[i].w;
    else es[u++] = es[i];
  }
  C->xadj = (int64_t*)fxalloc(nc + 1, sizeof(int64_t));
  C->adj = (int32_t*)fxalloc(u, sizeof(int32_t));
  C->w = (int32_t*)fxalloc(u, sizeof(int32_t));
  for (int64_t i = 0; i < u; i++) {
    C->xadj[es[i].a + 1]++;
    C->adj[i] = es[i].b;
    C->w[i] = (int32_t)es[i].w;
  }
  for (int64_t c = 0; c < nc; c++) C->xadj[c + 1] += C->xadj[c];
  free(es);
}

static int g_fgp_init = 0;
void ora_fgp_set_init(int v) { g_fgp_init = v; }
/* F5: greedy graph growing on the coarsest graph */
static void fgp_initial(const fcsr* G, int32_t k, int32_t* part) {
  if (g_fgp_init == 1) {  /* contiguous ID blocks by cumulative weight */
    int64_t W = 0, acc = 0;
    for (int64_t v = 0; v < G->n; v++) W += G->vw[v];
    int32_t p = 0;
    for (int64_t v = 0; v < G->n; v++) {
      part[v] = p;
      acc += G->vw[v];
      if (p < k - 1 && acc * k >= (int64_t)(p + 1) * W) p++;
    }
    return;
  }
  const int64_t n = G->n;
  int64_t W = 0;
  for (int64_t v = 0; v < n; v++) W += G->vw[v];
  uint8_t* vis = (uint8_t*)fxalloc(n, 1);
  int32_t* q = (int32_t*)fxalloc(n, sizeof(int32_t));
  int64_t acc = 0;
  int32_t p = 0;
  for (int64_t s = 0; s < n; s++) {
    if (vis[s]) continue;
    int64_t qh = 0, qt = 0;
    q[qt++] = (int32_t)s;
    vis[s] = 1;
    while (qh < qt) {
      const int32_t v = q[qh++];
      part[v] = p;
      acc += G->vw[v];
      if (p < k - 1 && acc * k >= (int64_t)(p + 1) * W) p++;
      for (int64_t j = G->xadj[v]; j < G->xadj[v + 1]; j++) {
        const int32_t x = G->adj[j];
        if (!vis[x]) {
          vis[x] = 1;
          q[qt++] = x;
        }
      }
    }
  }
  free(vis);
  free(q);
}

/* F6: refine a level's partition with the global boundary refinement,
 * repeated while a pass lowers the cut (at most kFgpPasses passes) */
static int g_fgp_passes = 8;
void ora_fgp_set_passes(int p) { g_fgp_passes = p; }
static int fgp_refine(const fcsr* G, int32_t k, double eps, int32_t* part) {
  int st = 0;
  ora_graph* g = ora_create_ex(G->n, G->xadj, G->adj, G->vw, G->w, k, eps, part, 1, &st);
  if (!g) return -1;
  int64_t stats[ORA_NSTATS];
  int64_t prev = -1;
  int rs = ORA_OK;
  for (int pass = 0; pass < g_fgp_passes; pass++) {
    rs = ora_refine_global(g, stats);
    if (rs != ORA_OK && rs != ORA_WIMBALANCED) break;
    if (prev >= 0 && stats[ORA_ST_CUT] >= prev) break;
    prev = stats[ORA_ST_CUT];
  }
  ora_partition(g, part);
  ora_destroy(g);
  return rs == ORA_OK || rs == ORA_WIMBALANCED ? 0 : -1;
}

/* F7: one synchronous label-propagation pass on a snapshot of part / W_p.
 *  a. every vertex v in part a: conn_p = sum of w(v, x) over neighbours x
 *     in part p; b = the part p != a of maximal conn_p, smallest p on ties,
 *     over the parts of v's neighbours; gain g_v = conn_b - conn_a; v is a
 *     candidate iff g_v > 0.
 *  b. a candidate moves only if it beats every candidate neighbour u in
 *     (g desc, ID asc) -- the movers are pairwise non-adjacent, so the cut
 *     falls by exactly the sum of their gains.
 *  c. balance: the movers into part b, in (g desc, ID asc) order, are
 *     admitted while W_b + (their running weight) <= cap (a prefix).
 * Returns the number of vertices moved; *dcut gets the cut reduction. */
static int g_lp_passes = 16;

void ora_fgp_set_lp_passes(int p) { g_lp_passes = p; }
typedef struct {
  int32_t b;
  int64_t g;
  int32_t id;
} lpmove;
static int cmp_lpmove(const void* x, const void* y) {
  const lpmove* p = (const lpmove*)x;
  const lpmove* q = (const lpmove*)y;
  if (p->b != q->b) return p->b < q->b ? -1 : 1;
  if (p->g != q->g) return p->g > q->g ? -1 : 1;
  return p->id < q->id ? -1 : (p->id > q->id);
}
static int64_t fgp_lp_pass(const fcsr* G, int32_t k, int64_t cap, int32_t* part, int64_t* W, int64_t* dcut) {
  const int64_t n = G->n;
  int64_t* conn = (int64_t*)fxalloc(k, sizeof(int64_t));
  int32_t* tgt = (int32_t*)fxalloc(n, sizeof(int32_t));
  int64_t* gain = (int64_t*)fxalloc(n, sizeof(int64_t));
  for (int64_t v = 0; v < n; v++) { /* a */
    const int32_t a = part[v];
    for (int32_t p = 0; p < k; p++) conn[p] = 0;
    for (int64_t j = G->xadj[v]; j < G->xadj[v + 1]; j++) conn[part[G->adj[j]]] += G->w[j];
    int32_t b = -1;
    for (int64_t j = G->xadj[v]; j < G->xadj[v + 1]; j++) {
      const int32_t p = part[G->adj[j]];
      if (p != a && (b < 0 || conn[p] > conn[b] || (conn[p] == conn[b] && p < b))) b = p;
    }
    tgt[v] = -1;
    if (b >= 0 && conn[b] - conn[a] > 0) {
      tgt[v] = b;
      gain[v] = conn[b] - conn[a];
    }
  }
  lpmove* mv = (lpmove*)fxalloc(n, sizeof(lpmove));
  int64_t nm = 0;
  for (int64_t v = 0; v < n; v++) { /* b */
    if (tgt[v] < 0) continue;
    int beaten = 0;
    for (int64_t j = G->xadj[v]; j < G->xadj[v + 1] && !beaten; j++) {
      const int32_t u = G->adj[j];
      if (tgt[u] >= 0 && (gain[u] > gain[v] || (gain[u] == gain[v] && u < v))) beaten = 1;
    }
    if (!beaten) {
      mv[nm].b = tgt[v];
      mv[nm].g = gain[v];
      mv[nm].id = (int32_t)v;
      nm++;
    }
  }
  qsort(mv, nm, sizeof(lpmove), cmp_lpmove);
  int64_t moved = 0, red = 0, run = 0;
  for (int64_t i = 0; i < nm; i++) { /* c: the admission uses the W_b of the snapshot */
    if (i == 0 || mv[i].b != mv[i - 1].b) run = 0;
    run += G->vw[mv[i].id];
    if (W[mv[i].b] + run > cap) continue;
    tgt[mv[i].id] = -2 - mv[i].b; /* admitted (applied below) */
  }
  for (int64_t v = 0; v < n; v++)
    if (tgt[v] <= -2) {
      const int32_t b = -2 - tgt[v];
      W[part[v]] -= G->vw[v];
      W[b] += G->vw[v];
      part[v] = b;
      red += gain[v];
      moved++;
    }
  free(conn);
  free(tgt);
  free(gain);
  free(mv);
  *dcut = red;
  return moved;
}

static void fgp_lp(const fcsr* G, int32_t k, double eps, int32_t* part) {
  int64_t Wt = 0;
  int64_t* W = (int64_t*)fxalloc(k, sizeof(int64_t));
  for (int64_t v = 0; v < G->n; v++) {
    Wt += G->vw[v];
    W[part[v]] += G->vw[v];
  }
  const int64_t cap = ora_cap(Wt, eps, k);
  for (int pass = 0; pass < g_lp_passes; pass++) {
    int64_t dc = 0;
    if (fgp_lp_pass(G, k, cap, part, W, &dc) == 0) break;
  }
  free(W);
}

int64_t ora_fgp_lp_pass(int64_t n, const int64_t* xadj, const int32_t* adjncy, const int32_t* vwgt,
                        const int32_t* adjwgt, int32_t k, double epsilon, int32_t* part, int64_t* dcut) {
  fcsr G;
  G.n = n;
  G.xadj = (int64_t*)xadj;
  G.adj = (int32_t*)adjncy;
  const int64_t m2 = xadj[n];
  G.w = (int32_t*)fxalloc(m2, sizeof(int32_t));
  G.vw = (int32_t*)fxalloc(n, sizeof(int32_t));
  for (int64_t j = 0; j < m2; j++) G.w[j] = adjwgt ? adjwgt[j] : 1;
  int64_t Wt = 0;
  for (int64_t v = 0; v < n; v++) Wt += (G.vw[v] = vwgt ? vwgt[v] : 1);
  int64_t* W = (int64_t*)fxalloc(k, sizeof(int64_t));
  for (int64_t v = 0; v < n; v++) W[part[v]] += G.vw[v];
  const int64_t moved = fgp_lp_pass(&G, k, ora_cap(Wt, epsilon, k), part, W, dcut);
  free(W);
  free(G.w);
  free(G.vw);
  return moved;
}

int ora_fgp(int64_t n, const int64_t* xadj, const int32_t* adjncy, const int32_t* vwgt, const int32_t* adjwgt,
            int32_t k, double epsilon, int32_t group_size, int32_t* part_out, int64_t* level_n, int64_t maxlev) {
  if (n < 1 || k < 2 || group_size < 2) return -ORA_EINVAL;
  enum { kMaxLevels = 32 };
  fcsr L[kMaxLevels + 1];
  int32_t* cmaps[kMaxLevels];
  memset(L, 0, sizeof L);
  /* level 0: a copy with explicit weights */
  const int64_t m2 = xadj[n];
  L[0].n = n;
  L[0].xadj = (int64_t*)fxalloc(n + 1, sizeof(int64_t));
  L[0].adj = (int32_t*)fxalloc(m2, sizeof(int32_t));
  L[0].w = (int32_t*)fxalloc(m2, sizeof(int32_t));
  L[0].vw = (int32_t*)fxalloc(n, sizeof(int32_t));
  memcpy(L[0].xadj, xadj, (n + 1) * sizeof(int64_t));
  memcpy(L[0].adj, adjncy, m2 * sizeof(int32_t));
  for (int64_t j = 0; j < m2; j++) L[0].w[j] = adjwgt ? adjwgt[j] : 1;
  for (int64_t v = 0; v < n; v++) L[0].vw[v] = vwgt ? vwgt[v] : 1;
  int nl = 0; /* index of the coarsest level */
  while (nl < kMaxLevels && L[nl].n >= 35 * (int64_t)k) {
    const fcsr* G = &L[nl];
    int32_t* sel = (int32_t*)fxalloc(G->n, sizeof(int32_t));
    int32_t* root = (int32_t*)fxalloc(G->n, sizeof(int32_t));
    int32_t* label = (int32_t*)fxalloc(G->n, sizeof(int32_t));
    int32_t* cmap = (int32_t*)fxalloc(G->n, sizeof(int32_t));
    fgp_select(G, sel);
    fgp_union(G, sel, root, label);
    int64_t co = 0;
    const int64_t nc = fgp_group(G, root, label, group_size, cmap, &co);
    free(sel);
    free(root);
    free(label);
    if (co * 10 < G->n * 9 || nc >= G->n) { /* fewer than 90% coarsenable / no progress */
      free(cmap);
      break;
    }
    fgp_contract(G, cmap, nc, &L[nl + 1]);
    cmaps[nl] = cmap;
    nl++;
  }
  for (int l = 0; l <= nl && l < maxlev; l++) level_n[l] = L[l].n;
  /* initial partition + refinement of the coarsest level, then project and refine down */
  int32_t* part = (int32_t*)fxalloc(L[nl].n, sizeof(int32_t));
  fgp_initial(&L[nl], k, part);
  int bad = fgp_refine(&L[nl], k, epsilon, part);
  for (int l = nl - 1; l >= 0 && !bad; l--) {
    int32_t* fine = (int32_t*)fxalloc(L[l].n, sizeof(int32_t));
    for (int64_t v = 0; v < L[l].n; v++) fine[v] = part[cmaps[l][v]];
    free(part);
    part = fine;
    fgp_lp(&L[l], k, epsilon, part);
  }
  if (!bad) memcpy(part_out, part, n * sizeof(int32_t));
  free(part);
  for (int l = 0; l < nl; l++) free(cmaps[l]);
  for (int l = 0; l <= nl; l++) fcsr_free(&L[l]);
  return bad ? -ORA_EINVAL : nl + 1;  /* number of levels (>= 1), or -ORA_EINVAL */
}

/* step-level hooks for the pins: one coarsening step of a CSR graph */
int64_t ora_fgp_coarsen_step(int64_t n, const int64_t* xadj, const int32_t* adjncy, const int32_t* adjwgt,
                             int32_t group_size, int32_t* sel, int32_t* root, int32_t* label, int32_t* cmap,
                             int64_t* coarsenable) {
  fcsr G;
  G.n = n;
  G.xadj = (int64_t*)xadj;
  G.adj = (int32_t*)adjncy;
  const int64_t m2 = xadj[n];
  G.w = (int32_t*)fxalloc(m2, sizeof(int32_t));
  for (int64_t j = 0; j < m2; j++) G.w[j] = adjwgt ? adjwgt[j] : 1;
  G.vw = NULL;
  fgp_select(&G, sel);
  fgp_union(&G, sel, root, label);
  const int64_t nc = fgp_group(&G, root, label, group_size, cmap, coarsenable);
  free(G.w);
  return nc;
}
