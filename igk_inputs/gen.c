/*
 * gen.c -- seeded synthetic inputs for iG-kway incremental refinement.
 *
 * Shared by the oracle tests and the CUDA path; it contains NONE of the
 * method's arithmetic (no partition, filter, gain, cut or balance logic).
 * It only produces:
 *   - circuit-netlist-shaped graphs (drivers with heavy-tailed fanout,
 *     sinks mostly near the driver in ID order), DESIGN.md section 6;
 *   - an initial k-way partition (METIS_PartGraphKway from the CUDA
 *     toolkit's libmetis_static.a, or contiguous ID blocks);
 *   - valid modifier streams (vertex/edge insert/delete),
 *     for which it keeps a mirror of the edge set so that each batch is
 *     valid against the current graph.
 * PRNG: splitmix64 seeding xoshiro256** (counter-free, deterministic).
 */
#include <math.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

/* ---------------- PRNG ---------------- */
typedef struct { uint64_t s[4]; } rng_t;
static uint64_t splitmix64(uint64_t* x) {
  uint64_t z = (*x += 0x9E3779B97F4A7C15ull);
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
static void rng_seed(rng_t* r, uint64_t seed) {
  uint64_t x = seed;
  for (int i = 0; i < 4; i++) r->s[i] = splitmix64(&x);
}
static inline uint64_t rotl(uint64_t x, int k) { return (x << k) | (x >> (64 - k)); }
static uint64_t rng_next(rng_t* r) {
  uint64_t* s = r->s;
  uint64_t res = rotl(s[1] * 5, 7) * 9;
  uint64_t t = s[1] << 17;
  s[2] ^= s[0]; s[3] ^= s[1]; s[1] ^= s[2]; s[0] ^= s[3];
  s[2] ^= t; s[3] = rotl(s[3], 45);
  return res;
}
static uint64_t rng_below(rng_t* r, uint64_t n) { /* unbiased enough for n << 2^64 */
  return n ? rng_next(r) % n : 0;
}
static double rng_unit(rng_t* r) { return (rng_next(r) >> 11) * (1.0 / 9007199254740992.0); }
/* geometric on {1,2,...} with mean ~ w */
static int64_t rng_geom(rng_t* r, double w) {
  double u = rng_unit(r);
  if (u <= 0) u = 1e-300;
  double p = 1.0 / w;
  int64_t g = (int64_t)floor(log(u) / log(1.0 - p)) + 1;
  return g < 1 ? 1 : g;
}

/* ---------------- dynamic adjacency mirror ---------------- */
typedef struct { int32_t* nb; int32_t* w; int32_t cnt, cap; } dadj;
static void dpush(dadj* a, int32_t x, int32_t w) {
  if (a->cnt == a->cap) {
    a->cap = a->cap ? a->cap * 2 : 4;
    a->nb = (int32_t*)realloc(a->nb, sizeof(int32_t) * a->cap);
    a->w = (int32_t*)realloc(a->w, sizeof(int32_t) * a->cap);
  }
  a->nb[a->cnt] = x; a->w[a->cnt] = w; a->cnt++;
}
static int dfind(const dadj* a, int32_t x) {
  for (int32_t i = 0; i < a->cnt; i++) if (a->nb[i] == x) return i;
  return -1;
}
static void dremove(dadj* a, int32_t x) {
  int i = dfind(a, x);
  if (i < 0) return;
  a->nb[i] = a->nb[a->cnt - 1]; a->w[i] = a->w[a->cnt - 1]; a->cnt--;
}

/* membership list with O(1) removal and uniform sampling */
typedef struct { int32_t* list; int32_t* pos; int64_t cnt, cap, pcap; } mset;
static void ms_reserve_pos(mset* m, int64_t n) {
  if (n <= m->pcap) return;
  int64_t c = m->pcap ? m->pcap : 16;
  while (c < n) c *= 2;
  m->pos = (int32_t*)realloc(m->pos, sizeof(int32_t) * c);
  for (int64_t i = m->pcap; i < c; i++) m->pos[i] = -1;
  m->pcap = c;
}
static void ms_add(mset* m, int32_t v) {
  ms_reserve_pos(m, (int64_t)v + 1);
  if (m->pos[v] >= 0) return;
  if (m->cnt == m->cap) {
    m->cap = m->cap ? m->cap * 2 : 16;
    m->list = (int32_t*)realloc(m->list, sizeof(int32_t) * m->cap);
  }
  m->pos[v] = (int32_t)m->cnt;
  m->list[m->cnt++] = v;
}
static int ms_has(const mset* m, int32_t v) { return v >= 0 && v < m->pcap && m->pos[v] >= 0; }
static void ms_del(mset* m, int32_t v) {
  if (!ms_has(m, v)) return;
  int32_t i = m->pos[v], last = m->list[m->cnt - 1];
  m->list[i] = last; m->pos[last] = i; m->cnt--; m->pos[v] = -1;
}

/* ---------------- graph generation ---------------- */
typedef struct {
  int64_t n;
  int64_t* xadj;
  int32_t* adjncy;
  int32_t* vwgt;
  int32_t* adjwgt;
} ggraph;

/* truncated discrete power law on [1, fmax] with mean 2 (alpha by bisection) */
static double* powerlaw_cdf(int64_t fmax, double mean) {
  double lo = 1.0001, hi = 6.0, alpha = 2.0;
  for (int it = 0; it < 200; it++) {
    alpha = 0.5 * (lo + hi);
    double z = 0, m = 0;
    for (int64_t f = 1; f <= fmax; f++) { double p = pow((double)f, -alpha); z += p; m += f * p; }
    if (m / z > mean) lo = alpha; else hi = alpha;
  }
  double* cdf = (double*)malloc(sizeof(double) * (fmax + 1));
  double z = 0;
  for (int64_t f = 1; f <= fmax; f++) z += pow((double)f, -alpha);
  double acc = 0;
  cdf[0] = 0;
  for (int64_t f = 1; f <= fmax; f++) { acc += pow((double)f, -alpha) / z; cdf[f] = acc; }
  cdf[fmax] = 1.0;
  return cdf;
}
static int64_t sample_cdf(const double* cdf, int64_t fmax, double u) {
  int64_t lo = 1, hi = fmax;
  while (lo < hi) { int64_t mid = (lo + hi) / 2; if (cdf[mid] < u) lo = mid + 1; else hi = mid; }
  return lo;
}

static int edge_exists(dadj* A, int32_t u, int32_t v) {
  return A[u].cnt <= A[v].cnt ? dfind(&A[u], v) >= 0 : dfind(&A[v], u) >= 0;
}

ggraph* gen_graph(int64_t n, int64_t fmax, int32_t window, double p_local, uint64_t seed,
                  int weighted) {
  rng_t r;
  rng_seed(&r, seed);
  double* cdf = powerlaw_cdf(fmax, 2.0);
  dadj* A = (dadj*)calloc(n, sizeof(dadj));
  for (int64_t u = 0; u < n; u++) {
    int64_t f = sample_cdf(cdf, fmax, rng_unit(&r));
    for (int64_t t = 0; t < f; t++) {
      for (int retry = 0; retry < 8; retry++) {
        int64_t v;
        if (rng_unit(&r) < p_local) {
          int64_t d = rng_geom(&r, window);
          v = (rng_next(&r) & 1) ? u + d : u - d;
        } else {
          v = (int64_t)rng_below(&r, n);
        }
        if (v < 0 || v >= n || v == u) continue;
        if (edge_exists(A, (int32_t)u, (int32_t)v)) continue;
        int32_t w = weighted ? (int32_t)(1 + rng_below(&r, 4)) : 1;
        dpush(&A[u], (int32_t)v, w);
        dpush(&A[v], (int32_t)u, w);
        break;
      }
    }
  }
  free(cdf);
  ggraph* g = (ggraph*)calloc(1, sizeof(ggraph));
  g->n = n;
  g->xadj = (int64_t*)malloc(sizeof(int64_t) * (n + 1));
  g->xadj[0] = 0;
  for (int64_t u = 0; u < n; u++) g->xadj[u + 1] = g->xadj[u] + A[u].cnt;
  int64_t m2 = g->xadj[n];
  g->adjncy = (int32_t*)malloc(sizeof(int32_t) * (m2 ? m2 : 1));
  g->adjwgt = (int32_t*)malloc(sizeof(int32_t) * (m2 ? m2 : 1));
  g->vwgt = (int32_t*)malloc(sizeof(int32_t) * (n ? n : 1));
  for (int64_t u = 0; u < n; u++) {
    memcpy(g->adjncy + g->xadj[u], A[u].nb, sizeof(int32_t) * A[u].cnt);
    memcpy(g->adjwgt + g->xadj[u], A[u].w, sizeof(int32_t) * A[u].cnt);
    g->vwgt[u] = weighted ? (int32_t)(1 + rng_below(&r, 4)) : 1;
    free(A[u].nb); free(A[u].w);
  }
  free(A);
  return g;
}
int64_t gg_n(const ggraph* g) { return g->n; }
int64_t gg_m2(const ggraph* g) { return g->xadj[g->n]; }
void gg_copy(const ggraph* g, int64_t* xadj, int32_t* adjncy, int32_t* vwgt, int32_t* adjwgt) {
  memcpy(xadj, g->xadj, sizeof(int64_t) * (g->n + 1));
  memcpy(adjncy, g->adjncy, sizeof(int32_t) * g->xadj[g->n]);
  memcpy(vwgt, g->vwgt, sizeof(int32_t) * g->n);
  memcpy(adjwgt, g->adjwgt, sizeof(int32_t) * g->xadj[g->n]);
}
void gg_free(ggraph* g) {
  if (!g) return;
  free(g->xadj); free(g->adjncy); free(g->vwgt); free(g->adjwgt); free(g);
}

/* ---------------- initial partition ---------------- */
typedef int64_t idx_t;
int METIS_PartGraphKway(idx_t*, idx_t*, idx_t*, idx_t*, idx_t*, idx_t*, idx_t*, idx_t*, void*, void*,
                        idx_t*, idx_t*, idx_t*);
int METIS_SetDefaultOptions(idx_t*);

/* METIS k-way with default options (ufactor 30 = 3% imbalance); returns
 * the METIS status (1 = OK) and the edge cut in *objval */
int gen_metis(int64_t n, const int64_t* xadj, const int32_t* adjncy, const int32_t* vwgt,
              const int32_t* adjwgt, int32_t k, int32_t* part, int64_t* objval) {
  idx_t nv = n, ncon = 1, np = k, obj = 0;
  idx_t opts[40];
  METIS_SetDefaultOptions(opts);
  int64_t m2 = xadj[n];
  idx_t* xa = (idx_t*)malloc(sizeof(idx_t) * (n + 1));
  idx_t* ad = (idx_t*)malloc(sizeof(idx_t) * (m2 ? m2 : 1));
  idx_t* vw = vwgt ? (idx_t*)malloc(sizeof(idx_t) * (n ? n : 1)) : NULL;
  idx_t* aw = adjwgt ? (idx_t*)malloc(sizeof(idx_t) * (m2 ? m2 : 1)) : NULL;
  idx_t* pp = (idx_t*)malloc(sizeof(idx_t) * (n ? n : 1));
  for (int64_t i = 0; i <= n; i++) xa[i] = xadj[i];
  for (int64_t i = 0; i < m2; i++) { ad[i] = adjncy[i]; if (aw) aw[i] = adjwgt[i]; }
  for (int64_t i = 0; i < n; i++) if (vw) vw[i] = vwgt[i];
  int st = METIS_PartGraphKway(&nv, &ncon, xa, ad, vw, NULL, aw, &np, NULL, NULL, opts, &obj, pp);
  for (int64_t i = 0; i < n; i++) part[i] = (int32_t)pp[i];
  *objval = obj;
  free(xa); free(ad); free(vw); free(aw); free(pp);
  return st;
}

/* ---------------- modifier streams ---------------- */
enum { K_ED = 0, K_VD = 1, K_VI = 2, K_EI = 3 };
enum { MODE_MIX = 0, MODE_LITERAL = 1, MODE_ADVERSARIAL = 2 };

typedef struct {
  rng_t r;
  int64_t n;       /* n_total (IDs ever used) */
  int64_t ncap;
  dadj* A;
  mset act;        /* active vertices */
  mset r0;         /* adversarial region */
  int weighted;
  int32_t window;
  double p_local;
  int32_t* mark;   /* per-vertex batch stamp */
  int32_t stamp;
  int64_t* bkeys;  /* edge keys used in the current batch (small open hash) */
  int64_t bcap;
  int32_t* out;    /* current batch, 4 int32 per modifier */
  int64_t ocnt, ocap;
  int64_t m;       /* undirected edges in the mirror */
} gstream;

static void gs_grow(gstream* s, int64_t need) {
  if (need <= s->ncap) return;
  int64_t c = s->ncap ? s->ncap : 16;
  while (c < need) c *= 2;
  s->A = (dadj*)realloc(s->A, sizeof(dadj) * c);
  s->mark = (int32_t*)realloc(s->mark, sizeof(int32_t) * c);
  for (int64_t i = s->ncap; i < c; i++) { memset(&s->A[i], 0, sizeof(dadj)); s->mark[i] = 0; }
  s->ncap = c;
}

gstream* gen_stream_create(int64_t n, const int64_t* xadj, const int32_t* adjncy,
                           const int32_t* adjwgt, const int32_t* region0 /* nullable flags */,
                           uint64_t seed, int weighted) {
  gstream* s = (gstream*)calloc(1, sizeof(gstream));
  rng_seed(&s->r, seed);
  s->window = 256;
  s->p_local = 0.9;
  s->weighted = weighted;
  gs_grow(s, n + 16);
  s->n = n;
  for (int64_t u = 0; u < n; u++) {
    for (int64_t j = xadj[u]; j < xadj[u + 1]; j++) dpush(&s->A[u], adjncy[j], adjwgt ? adjwgt[j] : 1);
    s->m += xadj[u + 1] - xadj[u];
    ms_add(&s->act, (int32_t)u);
    if (region0 && region0[u]) ms_add(&s->r0, (int32_t)u);
  }
  s->m /= 2;
  return s;
}

static void out_push(gstream* s, int32_t kd, int32_t u, int32_t v, int32_t w) {
  if (s->ocnt == s->ocap) {
    s->ocap = s->ocap ? s->ocap * 2 : 1024;
    s->out = (int32_t*)realloc(s->out, sizeof(int32_t) * 4 * s->ocap);
  }
  int32_t* o = s->out + 4 * s->ocnt++;
  o[0] = kd; o[1] = u; o[2] = v; o[3] = w;
}

/* batch-local edge key set (open addressing, cleared per batch) */
static void bk_reset(gstream* s, int64_t expect) {
  int64_t c = 64;
  while (c < 4 * expect) c *= 2;
  if (c > s->bcap) { free(s->bkeys); s->bkeys = (int64_t*)malloc(sizeof(int64_t) * c); s->bcap = c; }
  for (int64_t i = 0; i < s->bcap; i++) s->bkeys[i] = -1;
}
static int bk_insert(gstream* s, int32_t u, int32_t v) { /* 1 if newly inserted */
  int64_t a = u < v ? u : v, b = u < v ? v : u;
  int64_t key = a << 32 | b;
  uint64_t h = (uint64_t)key * 0x9E3779B97F4A7C15ull;
  int64_t i = (int64_t)(h >> 20) & (s->bcap - 1);
  while (s->bkeys[i] != -1) {
    if (s->bkeys[i] == key) return 0;
    i = (i + 1) & (s->bcap - 1);
  }
  s->bkeys[i] = key;
  return 1;
}

static int32_t pick_active(gstream* s) { return s->act.list[rng_below(&s->r, s->act.cnt)]; }

/* one batch.  mode MIX: B = round(frac * n_active / 1.8) modifiers, 10% VI
 * (each with 1-3 local EI from the EI budget), 10% VD, 40% ED, 40% EI.
 * mode LITERAL: exactly nvd VD, nvi VI, ned ED, nei EI (C1's "1% of edges
 * and vertices").  mode ADVERSARIAL: nvd VD inside region R0 and nvi VI
 * attached only to R0 (C5).  The mirror is updated with S1's phase order. */
int64_t gen_stream_next(gstream* s, int mode, double frac, int64_t nvd, int64_t nvi, int64_t ned,
                        int64_t nei) {
  s->ocnt = 0;
  s->stamp++;
  if (mode == MODE_MIX) {
    /* edge-conserving mix: B0 base modifiers, 10% VI, 10% VD,
     * 40% ED, and EI = the ED count PLUS the edges the batch's vertex
     * deletions remove, so the edge count (and, with VI = VD, the average
     * degree ~4 of the north_star's inputs) stays level over thousands of
     * iterations.  A base modifier touches 2.6 vertices on average (VI, VD
     * one each; ED and the doubled EI two each), so B0 = f n / 2.6 keeps
     * the batch at ~f n touched vertices (SURVEY 8(d)'s B = f n / 1.8 for
     * the draining 10/10/40/40 mix). */
    int64_t B = llround(frac * (double)s->act.cnt / 2.6);
    if (B < 10) B = 10;
    nvi = llround(0.1 * B); nvd = llround(0.1 * B); ned = llround(0.4 * B); nei = ned;
  }
  const int32_t st = s->stamp; /* mark[v] == st: deleted in this batch */
  const int64_t n0 = s->n;
  mset* pool = (mode == MODE_ADVERSARIAL) ? &s->r0 : &s->act;
  /* vertex deletions */
  int64_t got = 0;
  for (int64_t t = 0; got < nvd && t < 8 * nvd + 64 && pool->cnt > 1; t++) {
    int32_t u = pool->list[rng_below(&s->r, pool->cnt)];
    if (s->mark[u] == st) continue;
    s->mark[u] = st;
    out_push(s, K_VD, u, 0, 0);
    got++;
  }
  if (mode == MODE_MIX) { /* + the edges incident to the deleted vertices (each once) */
    for (int64_t i = 0; i < s->ocnt; i++) {
      const int32_t u = s->out[4 * i + 1];
      for (int32_t j = 0; j < s->A[u].cnt; j++) {
        const int32_t x = s->A[u].nb[j];
        if (s->mark[x] != st || x > u) nei++;
      }
    }
  }
  bk_reset(s, ned + nei + 3 * nvi + 16);
  /* edge deletions: random active vertex with edges, random neighbour */
  if (mode != MODE_ADVERSARIAL) {
    got = 0;
    for (int64_t t = 0; got < ned && t < 16 * ned + 64; t++) {
      int32_t u = pick_active(s);
      if (s->mark[u] == st || s->A[u].cnt == 0) continue;
      int32_t v = s->A[u].nb[rng_below(&s->r, s->A[u].cnt)];
      if (s->mark[v] == st) continue;
      if (!bk_insert(s, u, v)) continue;
      out_push(s, K_ED, u, v, 0);
      got++;
    }
  }
  /* vertex insertions with 1-3 local edges each */
  int64_t ei_used = 0;
  gs_grow(s, n0 + nvi + 16);
  for (int64_t j = 0; j < nvi; j++) {
    int32_t id = (int32_t)(n0 + j);
    int32_t w = s->weighted ? (int32_t)(1 + rng_below(&s->r, 4)) : 1;
    out_push(s, K_VI, 0, 0, w);
    int ne = 1 + (int)rng_below(&s->r, mode == MODE_LITERAL ? 2 : 3);
    if (mode != MODE_ADVERSARIAL && ne > nei - ei_used) ne = (int)(nei - ei_used);
    int32_t anchor = -1;
    for (int t = 0; t < 16 && anchor < 0; t++) {
      int32_t a = pool->list[rng_below(&s->r, pool->cnt)];
      if (s->mark[a] != st) anchor = a;
    }
    if (anchor < 0) continue;
    for (int e = 0; e < ne; e++) {
      int32_t v = anchor;
      if (e > 0) {
        if (mode == MODE_ADVERSARIAL) {
          v = pool->list[rng_below(&s->r, pool->cnt)];
        } else {
          int64_t d = rng_geom(&s->r, 8);
          int64_t c = (rng_next(&s->r) & 1) ? anchor + d : anchor - d;
          if (c < 0 || c >= n0) continue;
          v = (int32_t)c;
        }
      }
      if (!ms_has(&s->act, v) || s->mark[v] == st) continue;
      if (!bk_insert(s, id, v)) continue;
      int32_t ew = s->weighted ? (int32_t)(1 + rng_below(&s->r, 4)) : 1;
      out_push(s, K_EI, id, v, ew);
      ei_used++;
    }
  }
  /* remaining edge insertions among existing vertices (90% local) */
  if (mode != MODE_ADVERSARIAL) {
    int64_t want = nei - ei_used;
    got = 0;
    for (int64_t t = 0; got < want && t < 16 * want + 64; t++) {
      int32_t u = pick_active(s);
      if (s->mark[u] == st) continue;
      int64_t v;
      if (rng_unit(&s->r) < s->p_local) {
        int64_t d = rng_geom(&s->r, s->window);
        v = (rng_next(&s->r) & 1) ? u + d : u - d;
      } else {
        v = s->act.list[rng_below(&s->r, s->act.cnt)];
      }
      if (v < 0 || v >= n0 || v == u || !ms_has(&s->act, (int32_t)v) || s->mark[v] == st) continue;
      if (edge_exists(s->A, u, (int32_t)v)) continue;
      if (!bk_insert(s, u, (int32_t)v)) continue;
      int32_t ew = s->weighted ? (int32_t)(1 + rng_below(&s->r, 4)) : 1;
      out_push(s, K_EI, u, (int32_t)v, ew);
      got++;
    }
  }
  /* mirror update in S1 phase order: ED, VD, VI, EI */
  for (int64_t i = 0; i < s->ocnt; i++) {
    int32_t* o = s->out + 4 * i;
    if (o[0] == K_ED) { dremove(&s->A[o[1]], o[2]); dremove(&s->A[o[2]], o[1]); s->m--; }
  }
  for (int64_t i = 0; i < s->ocnt; i++) {
    int32_t* o = s->out + 4 * i;
    if (o[0] != K_VD) continue;
    int32_t u = o[1];
    for (int32_t j = 0; j < s->A[u].cnt; j++) dremove(&s->A[s->A[u].nb[j]], u);
    s->m -= s->A[u].cnt;
    s->A[u].cnt = 0;
    ms_del(&s->act, u);
    ms_del(&s->r0, u);
  }
  for (int64_t j = 0; j < nvi; j++) {
    ms_add(&s->act, (int32_t)(n0 + j));
    if (mode == MODE_ADVERSARIAL) ms_add(&s->r0, (int32_t)(n0 + j));
  }
  s->n = n0 + nvi;
  for (int64_t i = 0; i < s->ocnt; i++) {
    int32_t* o = s->out + 4 * i;
    if (o[0] == K_EI) { dpush(&s->A[o[1]], o[2], o[3]); dpush(&s->A[o[2]], o[1], o[3]); s->m++; }
  }
  return s->ocnt;
}
void gen_stream_copy(const gstream* s, int32_t* out) { memcpy(out, s->out, sizeof(int32_t) * 4 * s->ocnt); }
int64_t gen_stream_n_total(const gstream* s) { return s->n; }
int64_t gen_stream_n_active(const gstream* s) { return s->act.cnt; }
int64_t gen_stream_region_size(const gstream* s) { return s->r0.cnt; }
int64_t gen_stream_n_edges(const gstream* s) { return s->m; }
void gen_stream_free(gstream* s) {
  if (!s) return;
  for (int64_t i = 0; i < s->ncap; i++) { free(s->A[i].nb); free(s->A[i].w); }
  free(s->A); free(s->mark); free(s->bkeys); free(s->out);
  free(s->act.list); free(s->act.pos); free(s->r0.list); free(s->r0.pos);
  free(s);
}
