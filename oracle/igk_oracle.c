/*
 * igk_oracle.c -- plain, slow, single-threaded CPU oracle of IGK-SEM v1.
 *
 * TEST INFRASTRUCTURE ONLY (see igk_oracle.h).  Nothing in the product
 * path may include, link or call this file.
 *
 * Citations: "P:N" is line N of the paper text (PAPER.md of
 * dblp/paper_conf_dac_leejlczcshh25, "iG-kway: Incremental k-way Graph
 * Partitioning on GPU", DAC'25).  Readings of garbled / silent passages
 * are named G*, Q*, S*, R* and listed in DESIGN.md section 4.
 *
 * Data layout: one growable (neighbour, weight) array per vertex.  No
 * blocking, no fusion, no reordering beyond what the algorithm states.
 */
#include "igk_oracle.h"

#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>

#define PSI (-1) /* pseudo-partition label */
#define DEL (-2) /* deleted vertex (vertex_status = deleted) */

/* limits shared by specification with the product */
#define LIM_K_MAX 254
#define LIM_VW_MAX 65535
#define LIM_EW_MAX 255
#define LIM_DEG_MAX (1 << 23)
#define LIM_N_MAX (1 << 30)

typedef struct {
  int32_t* nb;
  int32_t* w;
  int32_t cnt, cap;
} ora_adj;

struct ora_graph {
  int64_t n, ncap;
  uint8_t* active;
  int32_t* vw;
  int32_t* part;
  ora_adj* adj;
  int32_t k;
  int64_t e_ppm;
  double eps;
  int vw_unit, ew_unit;
  int64_t W;
  int64_t Wp[LIM_K_MAX];
  uint8_t* inA; /* accumulated affected set A (Alg. 3 L7) */
  uint8_t* inF; /* vertices that entered Psi since the last refine (I4) */
  int32_t* prev_part; /* parts at the start of the last refine (I4) */
  int last_imbalanced;
  int wide;             /* NEXT-2 coarse level: wide weights, no modifiers */
  int64_t last_cap;
  /* trace of the last refine */
  int64_t ntrace, trace_cap;
  int64_t *trS, *trL;
  int64_t ntm, tm_cap; /* sorted moves of every round: (u, p, g) triples */
  int64_t* trM;
  uint8_t *trC1, *trC2, *trR3;
  char err[256];
};

/* ------------------------------------------------------------------ */
/* small helpers                                                       */
/* ------------------------------------------------------------------ */
static void* xcalloc(size_t n, size_t s) {
  void* p = calloc(n ? n : 1, s);
  if (!p) { fprintf(stderr, "oracle: out of memory\n"); abort(); }
  return p;
}
static void* xrealloc(void* p, size_t s) {
  void* q = realloc(p, s ? s : 1);
  if (!q) { fprintf(stderr, "oracle: out of memory\n"); abort(); }
  return q;
}

static void adj_push(ora_adj* a, int32_t x, int32_t w) {
  if (a->cnt == a->cap) {
    a->cap = a->cap ? 2 * a->cap : 4;
    a->nb = (int32_t*)xrealloc(a->nb, sizeof(int32_t) * a->cap);
    a->w = (int32_t*)xrealloc(a->w, sizeof(int32_t) * a->cap);
  }
  a->nb[a->cnt] = x;
  a->w[a->cnt] = w;
  a->cnt++;
}
/* position of x in adj(u), or -1 */
static int32_t adj_find(const ora_adj* a, int32_t x) {
  for (int32_t i = 0; i < a->cnt; i++)
    if (a->nb[i] == x) return i;
  return -1;
}
/* remove x from adj(u) (edge deletion: "find v in u's buckets and
 * mark v as empty"); order inside a list carries no meaning */
static void adj_remove(ora_adj* a, int32_t x) {
  int32_t i = adj_find(a, x);
  if (i < 0) return;
  a->nb[i] = a->nb[a->cnt - 1];
  a->w[i] = a->w[a->cnt - 1];
  a->cnt--;
}

static void grow_vertices(ora_graph* g, int64_t need) {
  if (need <= g->ncap) return;
  int64_t nc = g->ncap ? g->ncap : 16;
  while (nc < need) nc *= 2;
  g->active = (uint8_t*)xrealloc(g->active, nc);
  g->vw = (int32_t*)xrealloc(g->vw, sizeof(int32_t) * nc);
  g->part = (int32_t*)xrealloc(g->part, sizeof(int32_t) * nc);
  g->adj = (ora_adj*)xrealloc(g->adj, sizeof(ora_adj) * nc);
  g->inA = (uint8_t*)xrealloc(g->inA, nc);
  g->inF = (uint8_t*)xrealloc(g->inF, nc);
  g->prev_part = (int32_t*)xrealloc(g->prev_part, sizeof(int32_t) * nc);
  g->trC1 = (uint8_t*)xrealloc(g->trC1, nc);
  g->trC2 = (uint8_t*)xrealloc(g->trC2, nc);
  g->trR3 = (uint8_t*)xrealloc(g->trR3, nc);
  for (int64_t v = g->ncap; v < nc; v++) {
    g->active[v] = 0;
    g->vw[v] = 0;
    g->part[v] = DEL;
    memset(&g->adj[v], 0, sizeof(ora_adj));
    g->inA[v] = 0;
    g->inF[v] = 0;
    g->prev_part[v] = DEL;
    g->trC1[v] = g->trC2[v] = g->trR3[v] = 0;
  }
  g->ncap = nc;
}

/* ------------------------------------------------------------------ */
/* balance bound under reading Q4:                            */
/*   e = llround(eps * 1e6),                                            */
/*   cap(W) = max( floor(W (1e6 + e) / (1e6 k)), ceil(W / k) )          */
/* ------------------------------------------------------------------ */
static int64_t cap_of(int64_t W, int64_t e_ppm, int32_t k) {
  unsigned __int128 num = (unsigned __int128)(uint64_t)W * (uint64_t)(1000000 + e_ppm);
  unsigned __int128 den = (unsigned __int128)1000000 * (uint64_t)k;
  int64_t a = (int64_t)(num / den);
  int64_t b = (W + k - 1) / k;
  return a > b ? a : b;
}

int64_t ora_cap(int64_t W, double epsilon, int32_t k) {
  return cap_of(W, llround(epsilon * 1e6), k);
}

/* adj_int / adj_ext of u (P:48 definitions; Alg. 3 L16-21 counting,
 * read as weighted sums, reading Q1); computed on snapshot `snap` of the
 * partition array.  A pseudo neighbour is external (reading Q13). */
static void int_ext(const ora_graph* g, const int32_t* snap, int32_t u,
                    int64_t* in, int64_t* ex) {
  int64_t a = 0, b = 0;
  const ora_adj* L = &g->adj[u];
  for (int32_t i = 0; i < L->cnt; i++) {
    if (snap[L->nb[i]] == snap[u]) a += L->w[i];
    else b += L->w[i];
  }
  *in = a;
  *ex = b;
}

static int cmp_pair(const void* a, const void* b) {
  const int32_t* x = (const int32_t*)a;
  const int32_t* y = (const int32_t*)b;
  return x[0] < y[0] ? -1 : (x[0] > y[0]);
}

/* ------------------------------------------------------------------ */
/* create                                                              */
/* ------------------------------------------------------------------ */
/* wide = 1 (NEXT-2 coarse levels): vertex / edge weights up to INT32_MAX
 * with the totals bounded by INT32_MAX (so every per-vertex sum of the
 * method stays exact in 32 bits on the product side); such a graph accepts
 * no modifiers */
ora_graph* ora_create_ex(int64_t n, const int64_t* xadj, const int32_t* adjncy,
                         const int32_t* vwgt, const int32_t* adjwgt, int32_t k,
                         double epsilon, const int32_t* init_part, int wide, int* status) {
  const int64_t vw_max = wide ? INT32_MAX : LIM_VW_MAX, ew_max = wide ? INT32_MAX : LIM_EW_MAX;
  *status = ORA_EINVAL;
  if (n < 0 || n > LIM_N_MAX || k < 2 || k > LIM_K_MAX || !(epsilon > 0.0) ||
      !(epsilon <= 1.0) || (n > 0 && (!xadj || !init_part)))
    return NULL;
  if (xadj && xadj[0] != 0) return NULL;
  for (int64_t u = 0; u < n; u++) {
    if (xadj[u + 1] < xadj[u]) return NULL;
    if (init_part[u] < 0 || init_part[u] >= k) return NULL;
    if (vwgt && (vwgt[u] < 1 || vwgt[u] > vw_max)) return NULL;
    if (xadj[u + 1] - xadj[u] > LIM_DEG_MAX) return NULL;
  }
  ora_graph* g = (ora_graph*)xcalloc(1, sizeof(ora_graph));
  g->k = k;
  g->eps = epsilon;
  g->e_ppm = llround(epsilon * 1e6);
  g->vw_unit = vwgt == NULL;
  g->ew_unit = adjwgt == NULL;
  grow_vertices(g, n > 0 ? n : 1);
  g->n = n;
  for (int64_t u = 0; u < n; u++) {
    g->active[u] = 1;
    g->vw[u] = vwgt ? vwgt[u] : 1;
    g->part[u] = init_part[u];
    for (int64_t j = xadj[u]; j < xadj[u + 1]; j++) {
      int32_t x = adjncy[j];
      int32_t w = adjwgt ? adjwgt[j] : 1;
      if (x < 0 || x >= n || x == u || w < 1 || w > ew_max) {
        ora_destroy(g);
        return NULL;
      }
      adj_push(&g->adj[u], x, w);
    }
  }
  /* simple + symmetric with w_ux == w_xu: checked on sorted row copies */
  int64_t m2 = xadj[n];
  int32_t* rows = (int32_t*)xcalloc(2 * (size_t)m2, sizeof(int32_t));
  for (int64_t u = 0; u < n; u++) {
    int32_t* r = rows + 2 * xadj[u];
    const ora_adj* L = &g->adj[u];
    for (int32_t i = 0; i < L->cnt; i++) {
      r[2 * i] = L->nb[i];
      r[2 * i + 1] = L->w[i];
    }
    qsort(r, L->cnt, 2 * sizeof(int32_t), cmp_pair);
  }
  int okc = 1;
  for (int64_t u = 0; u < n && okc; u++) {
    const int32_t* r = rows + 2 * xadj[u];
    int64_t d = xadj[u + 1] - xadj[u];
    for (int64_t i = 0; i < d && okc; i++) {
      if (i > 0 && r[2 * i] == r[2 * i - 2]) okc = 0; /* duplicate */
      int32_t x = r[2 * i];
      const int32_t* rx = rows + 2 * xadj[x];
      int64_t lo = 0, hi = xadj[x + 1] - xadj[x];
      while (lo < hi) { /* binary search for u in row x */
        int64_t mid = (lo + hi) / 2;
        if (rx[2 * mid] < u) lo = mid + 1; else hi = mid;
      }
      if (lo >= xadj[x + 1] - xadj[x] || rx[2 * lo] != u || rx[2 * lo + 1] != r[2 * i + 1])
        okc = 0;
    }
  }
  free(rows);
  if (!okc) {
    ora_destroy(g);
    return NULL;
  }
  g->W = 0;
  for (int i = 0; i < k; i++) g->Wp[i] = 0;
  for (int64_t u = 0; u < n; u++) {
    g->W += g->vw[u];
    g->Wp[g->part[u]] += g->vw[u];
  }
  if (wide) {
    int64_t ew = 0;
    for (int64_t j = 0; j < m2; j++) ew += adjwgt ? adjwgt[j] : 1;
    if (g->W > INT32_MAX || ew / 2 > INT32_MAX) {
      ora_destroy(g);
      return NULL;
    }
    g->wide = 1;
  }
  g->last_cap = cap_of(g->W, g->e_ppm, k);
  *status = ORA_OK;
  return g;
}

ora_graph* ora_create(int64_t n, const int64_t* xadj, const int32_t* adjncy,
                      const int32_t* vwgt, const int32_t* adjwgt, int32_t k,
                      double epsilon, const int32_t* init_part, int* status) {
  return ora_create_ex(n, xadj, adjncy, vwgt, adjwgt, k, epsilon, init_part, 0, status);
}

void ora_destroy(ora_graph* g) {
  if (!g) return;
  for (int64_t v = 0; v < g->ncap; v++) {
    free(g->adj[v].nb);
    free(g->adj[v].w);
  }
  free(g->adj);
  free(g->active);
  free(g->vw);
  free(g->part);
  free(g->inA);
  free(g->inF);
  free(g->prev_part);
  free(g->trS);
  free(g->trL);
  free(g->trM);
  free(g->trC1);
  free(g->trC2);
  free(g->trR3);
  free(g);
}

const char* ora_last_error(const ora_graph* g) { return g ? g->err : "null handle"; }

/* ------------------------------------------------------------------ */
/* apply(batch): reading S1.                            */
/* Validation against the pre-batch state, then the four phases        */
/*   1 edge deletions, 2 vertex deletions (Alg. 2 L4-6, L11-13, */
/*   reading Q12), 3 vertex insertions (Alg. 2 L7-10; Alg. 3 L2-5),    */
/*   4 edge insertions (Alg. 1),                                       */
/* marking affected vertices as Alg. 3 L6-7 and P:182 state.           */
/* ------------------------------------------------------------------ */
typedef struct {
  int64_t key;
  int64_t idx;
} ekey;
static int cmp_ekey(const void* a, const void* b) {
  const ekey* x = (const ekey*)a;
  const ekey* y = (const ekey*)b;
  if (x->key != y->key) return x->key < y->key ? -1 : 1;
  return x->idx < y->idx ? -1 : (x->idx > y->idx);
}

int ora_apply(ora_graph* g, const int32_t* mods, int64_t count, int64_t* first_new_id,
              int64_t* bad_index) {
  if (first_new_id) *first_new_id = g->n;
  if (bad_index) *bad_index = -1;
  if (count < 0 || g->wide) return ORA_EINVAL;
  if (count == 0) return ORA_OK;
  const int64_t n = g->n;
  int64_t n_ins = 0;
  for (int64_t i = 0; i < count; i++)
    if (mods[4 * i] == 2) n_ins++;
  if (n + n_ins > LIM_N_MAX) {
    snprintf(g->err, sizeof g->err, "too many vertices");
    return ORA_EINVAL;
  }
  uint8_t* bad = (uint8_t*)xcalloc(count, 1);
  int32_t* ndel = (int32_t*)xcalloc(n, sizeof(int32_t));     /* VERTEX_DELETE count */
  int64_t* nins = (int64_t*)xcalloc(n + n_ins, sizeof(int64_t)); /* EDGE_INSERT count */
  for (int64_t i = 0; i < count; i++) {
    int32_t kd = mods[4 * i], u = mods[4 * i + 1];
    if (kd == 1 && u >= 0 && u < n) ndel[u]++;
  }
  /* duplicated undirected edges among all edge modifiers: every occurrence invalid */
  int64_t ne = 0;
  ekey* ek = (ekey*)xcalloc(count, sizeof(ekey));
  for (int64_t i = 0; i < count; i++) {
    int32_t kd = mods[4 * i], u = mods[4 * i + 1], v = mods[4 * i + 2];
    if (kd == 0 || kd == 3) {
      int64_t a = u < v ? u : v, b = u < v ? v : u;
      ek[ne].key = (int64_t)((uint64_t)(uint32_t)a << 32 | (uint32_t)b);
      ek[ne].idx = i;
      ne++;
      if (kd == 3) {
        if (u >= 0 && u < n + n_ins) nins[u]++;
        if (v >= 0 && v < n + n_ins) nins[v]++;
      }
    }
  }
  qsort(ek, ne, sizeof(ekey), cmp_ekey);
  for (int64_t j = 0; j + 1 < ne; j++)
    if (ek[j].key == ek[j + 1].key) bad[ek[j].idx] = bad[ek[j + 1].idx] = 1;
  free(ek);

#define OLD_LIVE(x) ((x) >= 0 && (x) < n && g->active[(x)] && ndel[(x)] == 0)
  for (int64_t i = 0; i < count; i++) {
    int32_t kd = mods[4 * i], u = mods[4 * i + 1], v = mods[4 * i + 2], w = mods[4 * i + 3];
    int ok = 1;
    if (kd == 0) { /* EDGE_DELETE: existing edge, endpoints not deleted in batch */
      ok = OLD_LIVE(u) && OLD_LIVE(v) && u != v && adj_find(&g->adj[u], v) >= 0;
    } else if (kd == 1) { /* VERTEX_DELETE: active vertex, at most once */
      ok = u >= 0 && u < n && g->active[u] && ndel[u] == 1;
    } else if (kd == 2) { /* VERTEX_INSERT: weight range */
      ok = g->vw_unit ? (w == 1) : (w >= 1 && w <= LIM_VW_MAX);
    } else if (kd == 3) { /* EDGE_INSERT */
      int uo = OLD_LIVE(u), vo = OLD_LIVE(v);
      int un = u >= n && u < n + n_ins, vn = v >= n && v < n + n_ins;
      ok = u != v && (uo || un) && (vo || vn);
      ok = ok && (g->ew_unit ? (w == 1) : (w >= 1 && w <= LIM_EW_MAX));
      if (ok && uo && vo) ok = adj_find(&g->adj[u], v) < 0;
      if (ok) {
        int64_t du = (u < n ? g->adj[u].cnt : 0) + nins[u];
        int64_t dv = (v < n ? g->adj[v].cnt : 0) + nins[v];
        ok = du <= LIM_DEG_MAX && dv <= LIM_DEG_MAX;
      }
    } else {
      ok = 0;
    }
    if (!ok) bad[i] = 1;
  }
#undef OLD_LIVE
  int64_t first_bad = -1;
  for (int64_t i = 0; i < count; i++)
    if (bad[i]) { first_bad = i; break; }
  free(bad);
  free(ndel);
  free(nins);
  if (first_bad >= 0) {
    if (bad_index) *bad_index = first_bad;
    snprintf(g->err, sizeof g->err, "invalid modifier at index %lld", (long long)first_bad);
    return ORA_EINVAL;
  }

  /* phase 1: edge deletions; A u= {u, v} (Alg. 3 L6-7) */
  for (int64_t i = 0; i < count; i++) {
    if (mods[4 * i] != 0) continue;
    int32_t u = mods[4 * i + 1], v = mods[4 * i + 2];
    adj_remove(&g->adj[u], v);
    adj_remove(&g->adj[v], u);
    g->inA[u] = g->inA[v] = 1;
  }
  /* phase 2: vertex deletions (Alg. 2 L4-6, L11-13; reading Q12: both
   * directions of every incident edge are removed); neighbours of the
   * deleted vertex are affected (P:182 case 2); W_p and W shrink */
  for (int64_t i = 0; i < count; i++) {
    if (mods[4 * i] != 1) continue;
    int32_t u = mods[4 * i + 1];
    ora_adj* L = &g->adj[u];
    for (int32_t j = 0; j < L->cnt; j++) {
      adj_remove(&g->adj[L->nb[j]], u);
      g->inA[L->nb[j]] = 1;
    }
    L->cnt = 0;
    if (g->part[u] >= 0) g->Wp[g->part[u]] -= g->vw[u];
    g->W -= g->vw[u];
    g->active[u] = 0;
    g->part[u] = DEL;
  }
  /* phase 3: vertex insertions (Alg. 2 L7-10): the j-th insertion gets
   * ID n + j; it goes to the pseudo-partition at once (Alg. 3 L2-5) */
  grow_vertices(g, n + n_ins);
  int64_t j = 0;
  for (int64_t i = 0; i < count; i++) {
    if (mods[4 * i] != 2) continue;
    int64_t id = n + j++;
    g->active[id] = 1;
    g->vw[id] = mods[4 * i + 3];
    g->part[id] = PSI;
    g->W += g->vw[id];
    g->inF[id] = 1;
    g->adj[id].cnt = 0;
  }
  g->n = n + n_ins;
  /* phase 4: edge insertions (Alg. 1); A u= {u, v} (Alg. 3 L6-7) */
  for (int64_t i = 0; i < count; i++) {
    if (mods[4 * i] != 3) continue;
    int32_t u = mods[4 * i + 1], v = mods[4 * i + 2], w = mods[4 * i + 3];
    adj_push(&g->adj[u], v, w);
    adj_push(&g->adj[v], u, w);
    g->inA[u] = g->inA[v] = 1;
  }
  /* A := A n active */
  for (int64_t v = 0; v < g->n; v++)
    if (!g->active[v]) g->inA[v] = 0;
  return ORA_OK;
}

/* ------------------------------------------------------------------ */
/* refine(): R1 filter, R2 expansion, R3 restoration, R4 rounds         */
/* ------------------------------------------------------------------ */
static void trace_push(ora_graph* g, int64_t S, int64_t L) {
  if (g->ntrace == g->trace_cap) {
    g->trace_cap = g->trace_cap ? 2 * g->trace_cap : 64;
    g->trS = (int64_t*)xrealloc(g->trS, sizeof(int64_t) * g->trace_cap);
    g->trL = (int64_t*)xrealloc(g->trL, sizeof(int64_t) * g->trace_cap);
  }
  g->trS[g->ntrace] = S;
  g->trL[g->ntrace] = L;
  g->ntrace++;
}

/* deferred commit of a candidate set to the pseudo-partition
 * (Alg. 3 L25-26; "deferring partition updates") */
static int64_t commit_to_psi(ora_graph* g, const uint8_t* cand, uint8_t* trace) {
  int64_t c = 0;
  for (int64_t u = 0; u < g->n; u++) {
    if (!cand[u]) continue;
    g->Wp[g->part[u]] -= g->vw[u];
    g->part[u] = PSI;
    g->inF[u] = 1;
    trace[u] = 1;
    c++;
  }
  return c;
}

typedef struct {
  int64_t loss; /* int(x) - ext(x) */
  int32_t id;
  int32_t vw;
} rkey;
static int cmp_rkey(const void* a, const void* b) {
  const rkey* x = (const rkey*)a;
  const rkey* y = (const rkey*)b;
  if (x->loss != y->loss) return x->loss < y->loss ? -1 : 1;
  return x->id < y->id ? -1 : (x->id > y->id);
}

typedef struct {
  int64_t g;  /* #nbr of m_u^{par,#nbr}, weighted (Q1) */
  int32_t u;
  int32_t p;
} omove;
/* sort by #nbr descending, ties by vertex ID ascending (Q5) */
static int cmp_move(const void* a, const void* b) {
  const omove* x = (const omove*)a;
  const omove* y = (const omove*)b;
  if (x->g != y->g) return x->g > y->g ? -1 : 1;
  return x->u < y->u ? -1 : (x->u > y->u);
}

int ora_refine(ora_graph* g, int64_t* stats) {
  const int64_t n = g->n;
  const int32_t k = g->k;
  int64_t st[ORA_NSTATS];
  memset(st, 0, sizeof st);
  g->ntrace = 0;
  g->ntm = 0;
  g->last_imbalanced = 0;
  const int64_t c = cap_of(g->W, g->e_ppm, k);
  g->last_cap = c;
  for (int64_t v = 0; v < n; v++) {
    g->prev_part[v] = g->part[v];
    g->inF[v] = 0; /* F restarts; inserted vertices have prev_part = PSI */
    g->trC1[v] = g->trC2[v] = g->trR3[v] = 0;
  }
  for (int64_t v = 0; v < n; v++) {
    if (!g->active[v]) continue;
    if (g->part[v] == PSI) st[ORA_ST_INSERTED]++;
    else if (g->inA[v]) st[ORA_ST_AFFECTED]++;
  }
  st[ORA_ST_AFFECTED] += st[ORA_ST_INSERTED];

  int32_t* snap = (int32_t*)xcalloc(n, sizeof(int32_t));
  uint8_t* cand = (uint8_t*)xcalloc(n, 1);

  /* R1 -- filter the affected vertices (Alg. 3 L8-24):
   * u in A, not pseudo, moves iff adj_ext > adj_int (strict, reading Q2),
   * all on snapshot sigma1; deferred commit (L25-26). */
  memcpy(snap, g->part, sizeof(int32_t) * n);
  for (int64_t u = 0; u < n; u++) {
    cand[u] = 0;
    if (!g->inA[u] || !g->active[u] || snap[u] == PSI) continue;
    int64_t in, ex;
    int_ext(g, snap, (int32_t)u, &in, &ex);
    if (ex > in) cand[u] = 1;
  }
  st[ORA_ST_FILTERED_IN] = commit_to_psi(g, cand, g->trC1);

  /* R2 -- expansion: every non-pseudo neighbour of a pseudo
   * vertex is marked affected and filtered with the same rule, on
   * snapshot sigma2; one hop only (reading Q7); deferred commit. */
  memcpy(snap, g->part, sizeof(int32_t) * n);
  uint8_t* inN = (uint8_t*)xcalloc(n, 1);
  for (int64_t u = 0; u < n; u++) {
    if (!g->active[u] || snap[u] != PSI) continue;
    const ora_adj* L = &g->adj[u];
    for (int32_t i = 0; i < L->cnt; i++)
      if (snap[L->nb[i]] != PSI) inN[L->nb[i]] = 1;
  }
  for (int64_t x = 0; x < n; x++) {
    cand[x] = 0;
    if (!inN[x]) continue;
    st[ORA_ST_EXPANDED]++;
    int64_t in, ex;
    int_ext(g, snap, (int32_t)x, &in, &ex);
    if (ex > in) cand[x] = 1;
  }
  free(inN);
  st[ORA_ST_EXPANDED_IN] = commit_to_psi(g, cand, g->trC2);

  /* R3 -- balance restoration (paper silent, reading Q9 / R3): for each
   * part i with W_i > c, order its vertices by (int - ext, id) ascending
   * on snapshot sigma3 and evict the shortest prefix whose weight is
   * >= W_i - c.  All parts' evictions are committed together. */
  memcpy(snap, g->part, sizeof(int32_t) * n);
  for (int64_t x = 0; x < n; x++) cand[x] = 0;
  for (int32_t i = 0; i < k; i++) {
    if (g->Wp[i] <= c) continue;
    int64_t m = 0;
    for (int64_t x = 0; x < n; x++)
      if (g->active[x] && snap[x] == i) m++;
    rkey* ks = (rkey*)xcalloc(m, sizeof(rkey));
    m = 0;
    for (int64_t x = 0; x < n; x++) {
      if (!g->active[x] || snap[x] != i) continue;
      int64_t in, ex;
      int_ext(g, snap, (int32_t)x, &in, &ex);
      ks[m].loss = in - ex;
      ks[m].id = (int32_t)x;
      ks[m].vw = g->vw[x];
      m++;
    }
    qsort(ks, m, sizeof(rkey), cmp_rkey);
    int64_t need = g->Wp[i] - c, acc = 0;
    for (int64_t j = 0; j < m && acc < need; j++) {
      cand[ks[j].id] = 1;
      acc += ks[j].vw;
    }
    free(ks);
  }
  st[ORA_ST_EVICTED] = commit_to_psi(g, cand, g->trR3);
  free(cand);
  free(snap);

  /* R4 -- parallel refinement rounds (Alg. 4), repeated until
   * the pseudo-partition is empty. */
  int32_t* psi = (int32_t*)xcalloc(n, sizeof(int32_t));
  int64_t npsi = 0;
  for (int64_t u = 0; u < n; u++)
    if (g->active[u] && g->part[u] == PSI) psi[npsi++] = (int32_t)u;
  omove* mv = (omove*)xcalloc(npsi, sizeof(omove));
  int64_t* conn = (int64_t*)xcalloc(k, sizeof(int64_t));
  int64_t run[LIM_K_MAX];
  int64_t Wr[LIM_K_MAX];
  while (npsi > 0) {
    /* round-start snapshot of W_p (reading Q14) */
    for (int32_t p = 0; p < k; p++) Wr[p] = g->Wp[p];
    int64_t ns = 0;
    for (int64_t j = 0; j < npsi; j++) {
      int32_t u = psi[j];
      const ora_adj* L = &g->adj[u];
      /* selection (Alg. 4 L5-10): u is selected iff it has no
       * neighbour in the pseudo-partition with a smaller vertex ID */
      int sel = 1;
      for (int32_t i = 0; i < L->cnt; i++)
        if (g->part[L->nb[i]] == PSI && L->nb[i] < u) { sel = 0; break; }
      if (!sel) continue;
      /* best part (Alg. 4 L11-20): count u's neighbours in
       * each part p (weighted, Q1); pseudo neighbours count for no part
       * (Q13); eligible p: W_p + W_u <= c (Q3); maximise
       * (conn, -W_p, -p) (Q6). */
      for (int32_t p = 0; p < k; p++) conn[p] = 0;
      for (int32_t i = 0; i < L->cnt; i++) {
        int32_t q = g->part[L->nb[i]];
        if (q >= 0) conn[q] += L->w[i];
      }
      int32_t best = -1;
      for (int32_t p = 0; p < k; p++) {
        if (Wr[p] + g->vw[u] > c) continue;
        if (best < 0 || conn[p] > conn[best] ||
            (conn[p] == conn[best] && Wr[p] < Wr[best]))
          best = p; /* ascending p: an equal (conn, W_p) keeps the lower p */
      }
      if (best < 0) { /* E(u) empty: weighted corner case (Q8) */
        best = 0;
        for (int32_t p = 1; p < k; p++)
          if (Wr[p] < Wr[best]) best = p;
        g->last_imbalanced = 1;
      }
      mv[ns].g = conn[best];
      mv[ns].u = u;
      mv[ns].p = best;
      ns++;
    }
    /* order: #nbr descending, vertex ID ascending (Q5) */
    qsort(mv, ns, sizeof(omove), cmp_move);
    /* balanced prefix (eq. P:202): delta_p_wgt accumulated per
     * part in move order; L = longest prefix with W_i + scan_i <= c for
     * every part i (Fig. 5); at least one move (Q8). */
    for (int32_t p = 0; p < k; p++) run[p] = 0;
    int64_t L = ns;
    for (int64_t j = 0; j < ns; j++) {
      run[mv[j].p] += g->vw[mv[j].u];
      if (Wr[mv[j].p] + run[mv[j].p] > c) { L = j; break; }
    }
    if (L == 0) {
      L = 1;
      g->last_imbalanced = 1;
    }
    for (int64_t j = 0; j < L; j++) {
      g->part[mv[j].u] = mv[j].p;
      g->Wp[mv[j].p] += g->vw[mv[j].u];
    }
    trace_push(g, ns, L);
    for (int64_t j = 0; j < ns; j++) {
      if (g->ntm + 3 > g->tm_cap) {
        g->tm_cap = g->tm_cap ? 2 * g->tm_cap : 192;
        g->trM = (int64_t*)xrealloc(g->trM, sizeof(int64_t) * g->tm_cap);
      }
      g->trM[g->ntm++] = mv[j].u;
      g->trM[g->ntm++] = mv[j].p;
      g->trM[g->ntm++] = mv[j].g;
    }
    st[ORA_ST_ROUNDS]++;
    st[ORA_ST_MOVES_APPLIED] += L;
    st[ORA_ST_MOVES_DEFERRED] += ns - L;
    /* Psi keeps ascending ID order */
    int64_t w = 0;
    for (int64_t j = 0; j < npsi; j++)
      if (g->part[psi[j]] == PSI) psi[w++] = psi[j];
    npsi = w;
  }
  free(conn);
  free(mv);
  free(psi);

  st[ORA_ST_CUT] = ora_cut(g);
  st[ORA_ST_CAP] = c;
  int64_t mx = 0;
  for (int32_t p = 0; p < k; p++)
    if (g->Wp[p] > mx) mx = g->Wp[p];
  st[ORA_ST_MAX_PART_WEIGHT] = mx;
  st[ORA_ST_IMBALANCED] = g->last_imbalanced;
  /* A := {} after the refine (F is kept for the I4 check) */
  for (int64_t v = 0; v < n; v++) g->inA[v] = 0;
  if (stats) memcpy(stats, st, sizeof st);
  return g->last_imbalanced ? ORA_WIMBALANCED : ORA_OK;
}

/* NEXT-1 global boundary refinement: G-kway's
 * refinement "refines all vertices on the partition boundary (i.e.,
 * vertices with adj_ext != 0)".  Reading B1: the boundary is
 * taken on the partition as it stands when the call is made (a pending
 * pseudo neighbour is external, reading Q13); every boundary vertex joins
 * the affected set A, then the ordinary refine runs (R1-R4 unchanged). */
int ora_refine_global(ora_graph* g, int64_t* stats) {
  for (int64_t u = 0; u < g->n; u++) {
    if (!g->active[u] || g->part[u] == PSI) continue;
    int64_t in, ex;
    int_ext(g, g->part, (int32_t)u, &in, &ex);
    if (ex != 0) g->inA[u] = 1;
  }
  return ora_refine(g, stats);
}

/* ------------------------------------------------------------------ */
/* queries                                                              */
/* ------------------------------------------------------------------ */
int64_t ora_n_total(const ora_graph* g) { return g->n; }
int64_t ora_n_active(const ora_graph* g) {
  int64_t c = 0;
  for (int64_t v = 0; v < g->n; v++) c += g->active[v];
  return c;
}
void ora_partition(const ora_graph* g, int32_t* out) {
  for (int64_t v = 0; v < g->n; v++)
    out[v] = !g->active[v] ? -1 : (g->part[v] == PSI ? -2 : g->part[v]);
}
/* cut size: sum of W_e over edges whose endpoints lie in
 * different parts; an edge with a pending (pseudo) endpoint is not
 * counted. */
int64_t ora_cut(const ora_graph* g) {
  int64_t c = 0;
  for (int64_t u = 0; u < g->n; u++) {
    if (!g->active[u] || g->part[u] < 0) continue;
    const ora_adj* L = &g->adj[u];
    for (int32_t i = 0; i < L->cnt; i++) {
      int32_t x = L->nb[i];
      if (x > u && g->part[x] >= 0 && g->part[x] != g->part[u]) c += L->w[i];
    }
  }
  return c;
}
void ora_part_weights(const ora_graph* g, int64_t* out) {
  for (int32_t p = 0; p < g->k; p++) out[p] = g->Wp[p];
}
int64_t ora_total_weight(const ora_graph* g) { return g->W; }
int64_t ora_cap_value(const ora_graph* g) { return cap_of(g->W, g->e_ppm, g->k); }

int64_t ora_num_slots(const ora_graph* g) {
  int64_t s = 0;
  for (int64_t v = 0; v < g->n; v++) s += g->adj[v].cnt;
  return s;
}
void ora_export_csr(const ora_graph* g, int64_t* xadj, int32_t* adjncy, int32_t* adjwgt) {
  int64_t pos = 0;
  xadj[0] = 0;
  for (int64_t v = 0; v < g->n; v++) {
    const ora_adj* L = &g->adj[v];
    int32_t* tmp = (int32_t*)xcalloc(2 * (size_t)L->cnt, sizeof(int32_t));
    for (int32_t i = 0; i < L->cnt; i++) {
      tmp[2 * i] = L->nb[i];
      tmp[2 * i + 1] = L->w[i];
    }
    qsort(tmp, L->cnt, 2 * sizeof(int32_t), cmp_pair);
    for (int32_t i = 0; i < L->cnt; i++) {
      adjncy[pos] = tmp[2 * i];
      if (adjwgt) adjwgt[pos] = tmp[2 * i + 1];
      pos++;
    }
    free(tmp);
    xadj[v + 1] = pos;
  }
}

/* invariants after a refine (north_star).  Checked in a
 * fixed order -- structure first, then labels, weights, balance, frontier,
 * cut -- and the first violation is reported with its tag:
 * I6 adjacency symmetric (equal weights both ways), simple, no self loops,
 *    no inactive endpoints (G = (V, E) undirected, simple)
 * I5 Psi empty: every active vertex has a part in [0,k) (rounds
 *    repeat until the pseudo-partition is empty)
 * I2 W = sum of active vw, every maintained W_p = its recount, sum W_p = W
 *    (P:48 part weights)
 * I3 W_p <= c for every part unless the weighted fallback fired
 * I4 only vertices that entered Psi in the last refine changed part
 *    (north_star "only frontier vertices moved")
 * I1 a caller-reported maintained cut equals the recount ora_cut;
 *    skipped when reported_cut < 0 (the oracle keeps no cut of its own)
 * I6 runs on sorted copies of every row: O(m log m), so it stays cheap on
 * 10^4-degree hubs (C4).  The recounts here share nothing with apply/refine. */
static int cmp_i32(const void* a, const void* b) {
  int32_t x = *(const int32_t*)a, y = *(const int32_t*)b;
  return x < y ? -1 : (x > y);
}
int ora_check_invariants_ext(const ora_graph* g, int64_t reported_cut, int flags, char* msg, int msglen) {
  const int64_t n = g->n;
  /* I6 (skipped with flags & 1: labels/weights only) ------------------ */
  if (!(flags & 1)) {
  int64_t* rs = (int64_t*)xcalloc((size_t)n + 1, sizeof(int64_t));
  for (int64_t v = 0; v < n; v++) rs[v + 1] = rs[v] + g->adj[v].cnt;
  int32_t* rows = (int32_t*)xcalloc(2 * (size_t)rs[n], sizeof(int32_t));
  for (int64_t v = 0; v < n; v++) {
    const ora_adj* L = &g->adj[v];
    int32_t* r = rows + 2 * rs[v];
    for (int32_t i = 0; i < L->cnt; i++) {
      r[2 * i] = L->nb[i];
      r[2 * i + 1] = L->w[i];
    }
    qsort(r, L->cnt, 2 * sizeof(int32_t), cmp_i32);
  }
  int bad = 0;
  for (int64_t v = 0; v < n && !bad; v++) {
    const int32_t* r = rows + 2 * rs[v];
    const int64_t d = rs[v + 1] - rs[v];
    if (!g->active[v]) {
      if (d) { snprintf(msg, msglen, "I6: deleted %lld has edges", (long long)v); bad = 1; }
      continue;
    }
    for (int64_t i = 0; i < d && !bad; i++) {
      const int32_t x = r[2 * i];
      if (x == v || x < 0 || x >= n || !g->active[x]) {
        snprintf(msg, msglen, "I6: bad neighbour %d of %lld", x, (long long)v);
        bad = 1;
        break;
      }
      if (i > 0 && r[2 * i - 2] == x) {
        snprintf(msg, msglen, "I6: duplicate edge %lld-%d", (long long)v, x);
        bad = 1;
        break;
      }
      const int32_t* rx = rows + 2 * rs[x];
      int64_t lo = 0, hi = rs[x + 1] - rs[x];
      while (lo < hi) { /* binary search for v in the sorted row of x */
        int64_t mid = (lo + hi) / 2;
        if (rx[2 * mid] < v) lo = mid + 1; else hi = mid;
      }
      if (lo >= rs[x + 1] - rs[x] || rx[2 * lo] != v || rx[2 * lo + 1] != r[2 * i + 1]) {
        snprintf(msg, msglen, "I6: asymmetric edge %lld-%d", (long long)v, x);
        bad = 1;
      }
    }
  }
  free(rows);
  free(rs);
  if (bad) return 1;
  }
  /* I5 ------------------------------------------------------------- */
  for (int64_t v = 0; v < n; v++) {
    if (!g->active[v]) continue;
    if (g->part[v] < 0 || g->part[v] >= g->k) {
      snprintf(msg, msglen, "I5: vertex %lld has part %d", (long long)v, g->part[v]);
      return 1;
    }
  }
  /* I2 ------------------------------------------------------------- */
  int64_t Wp[LIM_K_MAX];
  int64_t W = 0;
  for (int32_t p = 0; p < g->k; p++) Wp[p] = 0;
  for (int64_t v = 0; v < n; v++) {
    if (!g->active[v]) continue;
    W += g->vw[v];
    Wp[g->part[v]] += g->vw[v];
  }
  if (W != g->W) { snprintf(msg, msglen, "I2: W mismatch"); return 1; }
  int64_t s = 0;
  for (int32_t p = 0; p < g->k; p++) {
    s += g->Wp[p];
    if (Wp[p] != g->Wp[p]) { snprintf(msg, msglen, "I2: W_%d mismatch", p); return 1; }
  }
  if (s != g->W) { snprintf(msg, msglen, "I2: sum W_p != W"); return 1; }
  /* I3 ------------------------------------------------------------- */
  const int64_t c = cap_of(g->W, g->e_ppm, g->k);
  for (int32_t p = 0; p < g->k; p++)
    if (g->Wp[p] > c && !g->last_imbalanced) {
      snprintf(msg, msglen, "I3: W_%d=%lld > cap %lld", p, (long long)g->Wp[p], (long long)c);
      return 1;
    }
  /* I4 ------------------------------------------------------------- */
  for (int64_t v = 0; v < n; v++) {
    if (!g->active[v]) continue;
    if (!g->inF[v] && g->prev_part[v] >= 0 && g->prev_part[v] != g->part[v]) {
      snprintf(msg, msglen, "I4: vertex %lld moved outside the frontier", (long long)v);
      return 1;
    }
  }
  /* I1 ------------------------------------------------------------- */
  if (reported_cut >= 0) {
    int64_t rc = ora_cut(g);
    if (rc != reported_cut) {
      snprintf(msg, msglen, "I1: maintained cut %lld != recount %lld", (long long)reported_cut, (long long)rc);
      return 1;
    }
  }
  return 0;
}
int ora_check_invariants(const ora_graph* g, char* msg, int msglen) {
  return ora_check_invariants_ext(g, -1, 0, msg, msglen);
}

/* ------------------------------------------------------------------ */
/* TEST-ONLY corruption hooks: they write one field of the state so that */
/* tests can build states that violate exactly one invariant and check    */
/* that ora_check_invariants_ext names it.  They are never called by      */
/* apply/refine and carry none of the method's arithmetic.                */
/* ------------------------------------------------------------------ */
void ora_debug_set_part(ora_graph* g, int64_t v, int32_t p) { g->part[v] = p < 0 ? PSI : p; }
void ora_debug_set_part_weight(ora_graph* g, int32_t p, int64_t w) { g->Wp[p] = w; }
void ora_debug_set_total_weight(ora_graph* g, int64_t W) { g->W = W; }
void ora_debug_set_frontier(ora_graph* g, int64_t v, int f) { g->inF[v] = (uint8_t)(f != 0); }
void ora_debug_add_half_edge(ora_graph* g, int64_t u, int32_t x, int32_t w) { adj_push(&g->adj[u], x, w); }
void ora_debug_set_edge_weight(ora_graph* g, int64_t u, int32_t x, int32_t w) {
  int32_t i = adj_find(&g->adj[u], x);
  if (i >= 0) g->adj[u].w[i] = w;
}

int64_t ora_trace_rounds(const ora_graph* g, int64_t* S, int64_t* L, int64_t maxr) {
  for (int64_t r = 0; r < g->ntrace && r < maxr; r++) {
    S[r] = g->trS[r];
    L[r] = g->trL[r];
  }
  return g->ntrace;
}
void ora_trace_sets(const ora_graph* g, uint8_t* c1, uint8_t* c2, uint8_t* r3) {
  memcpy(c1, g->trC1, g->n);
  memcpy(c2, g->trC2, g->n);
  memcpy(r3, g->trR3, g->n);
}

int64_t ora_trace_moves(const ora_graph* g, int64_t* out, int64_t cap3) {
  for (int64_t i = 0; i < g->ntm && i < cap3; i++) out[i] = g->trM[i];
  return g->ntm / 3;
}

/* NEXT-2 full repartition, reading F8 (see igk_oracle.h) */
int ora_repartition(ora_graph* g, int32_t group_size) {
  const int64_t n = g->n;
  for (int64_t v = 0; v < n; v++)
    if (g->active[v] && (g->inA[v] || g->part[v] == PSI)) return ORA_ESTATE;
  int32_t* did = (int32_t*)xcalloc((size_t)n, sizeof(int32_t));
  int64_t na = 0, m2 = 0;
  for (int64_t v = 0; v < n; v++)
    if (g->active[v]) {
      did[v] = (int32_t)na++;
      m2 += g->adj[v].cnt;
    }
  if (na == 0) {
    free(did);
    return ORA_EINVAL;
  }
  int64_t* xadj = (int64_t*)xcalloc((size_t)na + 1, sizeof(int64_t));
  int32_t* adj = (int32_t*)xcalloc((size_t)m2, sizeof(int32_t));
  int32_t* w = (int32_t*)xcalloc((size_t)m2, sizeof(int32_t));
  int32_t* vw = (int32_t*)xcalloc((size_t)na, sizeof(int32_t));
  int32_t* part = (int32_t*)xcalloc((size_t)na, sizeof(int32_t));
  int64_t pos = 0;
  for (int64_t v = 0; v < n; v++) {
    if (!g->active[v]) continue;
    const ora_adj* L = &g->adj[v];
    int32_t* tmp = (int32_t*)xcalloc(2 * (size_t)L->cnt, sizeof(int32_t));
    for (int32_t i = 0; i < L->cnt; i++) {
      tmp[2 * i] = did[L->nb[i]]; /* dense IDs keep the ID order */
      tmp[2 * i + 1] = L->w[i];
    }
    qsort(tmp, L->cnt, 2 * sizeof(int32_t), cmp_pair);
    for (int32_t i = 0; i < L->cnt; i++) {
      adj[pos] = tmp[2 * i];
      w[pos] = tmp[2 * i + 1];
      pos++;
    }
    free(tmp);
    vw[did[v]] = g->vw[v];
    xadj[did[v] + 1] = pos;
  }
  int64_t lv[40];
  const int r = ora_fgp(na, xadj, adj, vw, w, g->k, g->eps, group_size, part, lv, 40);
  if (r >= 1) {
    for (int32_t p = 0; p < g->k; p++) g->Wp[p] = 0;
    for (int64_t v = 0; v < n; v++) {
      if (!g->active[v]) continue;
      g->part[v] = part[did[v]];
      g->Wp[g->part[v]] += g->vw[v];
      g->prev_part[v] = g->part[v];
      g->inF[v] = 0;
    }
  }
  free(did);
  free(xadj);
  free(adj);
  free(w);
  free(vw);
  free(part);
  return r >= 1 ? ORA_OK : ORA_EINVAL;
}
