/*
 * Plain C oracle for the MEGA GAT hot path — TEST INFRASTRUCTURE ONLY.
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load this.  Shares no code with the product.
 *
 * The same definitions as oracle/gat.py and oracle/traverse.py, written as
 * per-edge loops in fp64 (OpenMP over destinations / sources) so that full
 * BASELINE.json sizes finish in seconds.  Every function cites its passage:
 *   ora_gat_fwd      SURVEY §8(c)-c3; north_star e_ij.
 *   ora_gat_bwd      SURVEY §8(c)-c4 (closed form of the fwd's gradient).
 *   ora_*_rows/srcs  the same formulas restricted to sampled rows/sources.
 *   ora_traverse     reading R of Algorithm 1
 *                    (R8-R19).
 * Graph arguments: CSR by destination, indptr int64 [n+1], indices int32 [m].
 * Feature arguments: float [n][H*F] (the stored values, upcast to double).
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

static inline double leaky(double z, double slope) { return z > 0 ? z : slope * z; }

static void halves(int64_t n, int H, int F, const float *Wh, const float *a_l, const float *a_r,
                   double *el, double *er) {
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n; ++i)
    for (int h = 0; h < H; ++h) {
      double sl = 0, sr = 0;
      for (int f = 0; f < F; ++f) {
        double w = Wh[i * H * F + h * F + f];
        sl += (double)a_l[h * F + f] * w;
        sr += (double)a_r[h * F + f] * w;
      }
      el[i * H + h] = sl;
      er[i * H + h] = sr;
    }
}

/* one destination row, two-pass softmax (c3) */
static void fwd_row(int64_t i, const int64_t *indptr, const int32_t *indices, int H, int F, const float *Wh,
                    const float *a_r, double slope, const double *el_i, const double *er /* may be NULL */,
                    double *out_i, double *lse_i) {
  const int D = H * F;
  for (int d = 0; d < D; ++d) out_i[d] = 0;
  int64_t b = indptr[i], e = indptr[i + 1];
  for (int h = 0; h < H; ++h) {
    if (b == e) { lse_i[h] = -INFINITY; continue; }
    double m = -INFINITY;
    for (int64_t k = b; k < e; ++k) {
      int64_t j = indices[k];
      double erj;
      if (er) erj = er[j * H + h];
      else { erj = 0; for (int f = 0; f < F; ++f) erj += (double)a_r[h * F + f] * Wh[j * D + h * F + f]; }
      double s = leaky(el_i[h] + erj, slope);
      if (s > m) m = s;
    }
    double S = 0;
    for (int64_t k = b; k < e; ++k) {
      int64_t j = indices[k];
      double erj;
      if (er) erj = er[j * H + h];
      else { erj = 0; for (int f = 0; f < F; ++f) erj += (double)a_r[h * F + f] * Wh[j * D + h * F + f]; }
      S += exp(leaky(el_i[h] + erj, slope) - m);
    }
    for (int64_t k = b; k < e; ++k) {
      int64_t j = indices[k];
      double erj;
      if (er) erj = er[j * H + h];
      else { erj = 0; for (int f = 0; f < F; ++f) erj += (double)a_r[h * F + f] * Wh[j * D + h * F + f]; }
      double alpha = exp(leaky(el_i[h] + erj, slope) - m) / S;
      for (int f = 0; f < F; ++f) out_i[h * F + f] += alpha * Wh[j * D + h * F + f];
    }
    lse_i[h] = m + log(S);
  }
}

/* Full forward: out [n][D], lse/el/er [n][H] (double). */
void ora_gat_fwd(int64_t n, const int64_t *indptr, const int32_t *indices, int H, int F, const float *Wh,
                 const float *a_l, const float *a_r, double slope, double *out, double *lse, double *el,
                 double *er) {
  halves(n, H, F, Wh, a_l, a_r, el, er);
#pragma omp parallel for schedule(dynamic, 64)
  for (int64_t i = 0; i < n; ++i)
    fwd_row(i, indptr, indices, H, F, Wh, a_r, slope, el + i * H, er, out + i * (int64_t)H * F, lse + i * H);
}

/* Forward restricted to the listed destination rows: out [nr][D], lse [nr][H]. */
void ora_gat_fwd_rows(int64_t n, const int64_t *indptr, const int32_t *indices, int H, int F, const float *Wh,
                      const float *a_l, const float *a_r, double slope, int64_t nr, const int64_t *rows,
                      double *out, double *lse) {
  (void)n;
#pragma omp parallel for schedule(dynamic, 1)
  for (int64_t r = 0; r < nr; ++r) {
    int64_t i = rows[r];
    double el_i[64];
    const int D = H * F;
    for (int h = 0; h < H; ++h) {
      double s = 0;
      for (int f = 0; f < F; ++f) s += (double)a_l[h * F + f] * Wh[i * D + h * F + f];
      el_i[h] = s;
    }
    fwd_row(i, indptr, indices, H, F, Wh, a_r, slope, el_i, NULL, out + r * (int64_t)D, lse + r * H);
  }
}

/*
 * Full backward (c4).  Inputs: the forward's out/lse/el/er (double) and
 * grad_out g (float [n][D]).  Outputs (double): grad_feat [n][D],
 * grad_al/grad_ar [H][F], del/der [n][H].
 */
void ora_gat_bwd(int64_t n, const int64_t *indptr, const int32_t *indices, int H, int F, const float *Wh,
                 const float *a_l, const float *a_r, double slope, const float *g, const double *out,
                 const double *lse, const double *el, const double *er, double *grad_feat, double *grad_al,
                 double *grad_ar, double *del, double *der) {
  const int D = H * F;
  const int64_t m = indptr[n];
  double *Dlt = (double *)malloc(sizeof(double) * (size_t)(n * H));
  double *dz = (double *)malloc(sizeof(double) * (size_t)(m * H));
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n; ++i)
    for (int h = 0; h < H; ++h) {
      double s = 0;
      for (int f = 0; f < F; ++f) s += (double)g[i * D + h * F + f] * out[i * D + h * F + f];
      Dlt[i * H + h] = s;                                   /* Dlt_i = g_i . out_i */
    }
#pragma omp parallel for schedule(dynamic, 64)
  for (int64_t i = 0; i < n; ++i)
    for (int h = 0; h < H; ++h) {
      double acc = 0;
      for (int64_t k = indptr[i]; k < indptr[i + 1]; ++k) {
        int64_t j = indices[k];
        double z = el[i * H + h] + er[j * H + h];
        double alpha = exp(leaky(z, slope) - lse[i * H + h]);
        double da = 0;
        for (int f = 0; f < F; ++f) da += (double)g[i * D + h * F + f] * Wh[j * D + h * F + f];
        double ds = alpha * (da - Dlt[i * H + h]);
        double d = ds * (z > 0 ? 1.0 : slope);
        dz[k * H + h] = d;
        acc += d;
      }
      del[i * H + h] = acc;                                 /* del_i = sum_In dz */
    }
  /* source-major: CSC by counting sort */
  int64_t *cptr = (int64_t *)calloc((size_t)n + 1, sizeof(int64_t));
  int64_t *cedge = (int64_t *)malloc(sizeof(int64_t) * (size_t)(m > 0 ? m : 1));
  int64_t *cdst = (int64_t *)malloc(sizeof(int64_t) * (size_t)(m > 0 ? m : 1));
  for (int64_t k = 0; k < m; ++k) cptr[indices[k] + 1]++;
  for (int64_t v = 0; v < n; ++v) cptr[v + 1] += cptr[v];
  int64_t *fill = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n > 0 ? n : 1));
  memcpy(fill, cptr, sizeof(int64_t) * (size_t)n);
  for (int64_t i = 0; i < n; ++i)
    for (int64_t k = indptr[i]; k < indptr[i + 1]; ++k) { cedge[fill[indices[k]]] = k; cdst[fill[indices[k]]++] = i; }
  free(fill);
#pragma omp parallel for schedule(dynamic, 64)
  for (int64_t j = 0; j < n; ++j) {
    for (int d = 0; d < D; ++d) grad_feat[j * D + d] = 0;
    for (int h = 0; h < H; ++h) {
      double dr = 0;
      for (int64_t c = cptr[j]; c < cptr[j + 1]; ++c) {
        int64_t k = cedge[c], i = cdst[c];
        double alpha = exp(leaky(el[i * H + h] + er[j * H + h], slope) - lse[i * H + h]);
        for (int f = 0; f < F; ++f) grad_feat[j * D + h * F + f] += alpha * g[i * D + h * F + f];
        dr += dz[k * H + h];
      }
      der[j * H + h] = dr;                                  /* der_j = sum_Out dz */
      for (int f = 0; f < F; ++f)
        grad_feat[j * D + h * F + f] += dr * a_r[h * F + f] + del[j * H + h] * a_l[h * F + f];
    }
  }
  for (int d = 0; d < D; ++d) { grad_al[d] = 0; grad_ar[d] = 0; }
  for (int64_t i = 0; i < n; ++i)
    for (int h = 0; h < H; ++h)
      for (int f = 0; f < F; ++f) {
        grad_al[h * F + f] += del[i * H + h] * Wh[i * D + h * F + f];
        grad_ar[h * F + f] += der[i * H + h] * Wh[i * D + h * F + f];
      }
  free(cptr); free(cedge); free(cdst); free(Dlt); free(dz);
}

/*
 * grad_feat restricted to sampled sources js[ns] (c4's dWh_j line).  Needs, for
 * every out-edge (j -> i), row i's forward and Dlt_i; and del_j (row j's
 * in-edges).  Rows are recomputed on demand; O(sum of touched degrees * D).
 */
void ora_gat_bwd_srcs(int64_t n, const int64_t *indptr, const int32_t *indices, int H, int F, const float *Wh,
                      const float *a_l, const float *a_r, double slope, const float *g, int64_t ns,
                      const int64_t *js, double *grad_feat /* [ns][D] */) {
  const int D = H * F;
  const int64_t m = indptr[n];
  /* out-edge lists: dst of each edge, grouped by source */
  int64_t *cptr = (int64_t *)calloc((size_t)n + 1, sizeof(int64_t));
  int64_t *cdst = (int64_t *)malloc(sizeof(int64_t) * (size_t)(m > 0 ? m : 1));
  for (int64_t k = 0; k < m; ++k) cptr[indices[k] + 1]++;
  for (int64_t v = 0; v < n; ++v) cptr[v + 1] += cptr[v];
  int64_t *fill = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n > 0 ? n : 1));
  memcpy(fill, cptr, sizeof(int64_t) * (size_t)n);
  for (int64_t i = 0; i < n; ++i)
    for (int64_t k = indptr[i]; k < indptr[i + 1]; ++k) cdst[fill[indices[k]]++] = i;
  free(fill);
#pragma omp parallel for schedule(dynamic, 1)
  for (int64_t s = 0; s < ns; ++s) {
    int64_t j = js[s];
    double *gf = grad_feat + s * D;
    double *o = (double *)malloc(sizeof(double) * (size_t)D);
    double lse_i[64], el_i[64], Dlt_i[64], erj[64];
    for (int h = 0; h < H; ++h) {
      double t = 0;
      for (int f = 0; f < F; ++f) t += (double)a_r[h * F + f] * Wh[j * D + h * F + f];
      erj[h] = t;
    }
    for (int d = 0; d < D; ++d) gf[d] = 0;
    double der_j[64], del_j[64];
    for (int h = 0; h < H; ++h) { der_j[h] = 0; del_j[h] = 0; }
    /* rows whose dz we need: every out-neighbour i (for der_j, alpha g_i) and j itself (del_j) */
    for (int64_t c = cptr[j]; c <= cptr[j + 1]; ++c) {
      int self = (c == cptr[j + 1]);
      int64_t i = self ? j : cdst[c];
      for (int h = 0; h < H; ++h) {
        double t = 0;
        for (int f = 0; f < F; ++f) t += (double)a_l[h * F + f] * Wh[i * D + h * F + f];
        el_i[h] = t;
      }
      fwd_row(i, indptr, indices, H, F, Wh, a_r, slope, el_i, NULL, o, lse_i);
      for (int h = 0; h < H; ++h) {
        double t = 0;
        for (int f = 0; f < F; ++f) t += (double)g[i * D + h * F + f] * o[h * F + f];
        Dlt_i[h] = t;
      }
      if (!self) {
        /* this edge (j -> i): alpha, dz */
        for (int h = 0; h < H; ++h) {
          double z = el_i[h] + erj[h];
          double alpha = exp(leaky(z, slope) - lse_i[h]);
          double da = 0;
          for (int f = 0; f < F; ++f) da += (double)g[i * D + h * F + f] * Wh[j * D + h * F + f];
          der_j[h] += alpha * (da - Dlt_i[h]) * (z > 0 ? 1.0 : slope);
          for (int f = 0; f < F; ++f) gf[h * F + f] += alpha * g[i * D + h * F + f];
        }
      } else {
        /* del_j = sum over in-edges of j */
        for (int64_t k = indptr[j]; k < indptr[j + 1]; ++k) {
          int64_t q = indices[k];
          for (int h = 0; h < H; ++h) {
            double erq = 0, da = 0;
            for (int f = 0; f < F; ++f) {
              erq += (double)a_r[h * F + f] * Wh[q * D + h * F + f];
              da += (double)g[j * D + h * F + f] * Wh[q * D + h * F + f];
            }
            double z = el_i[h] + erq;
            double alpha = exp(leaky(z, slope) - lse_i[h]);
            del_j[h] += alpha * (da - Dlt_i[h]) * (z > 0 ? 1.0 : slope);
          }
        }
      }
    }
    for (int h = 0; h < H; ++h)
      for (int f = 0; f < F; ++f) gf[h * F + f] += der_j[h] * a_r[h * F + f] + del_j[h] * a_l[h * F + f];
    free(o);
  }
  free(cptr); free(cdst);
}

/* ---------------------------------------------------------------------------
 * Traversal R (R8-R19).  Plain: adjacency lists of G_u built by
 * counting, sorted and deduplicated; candidates scanned from a per-node cursor
 * that skips the leading visited entries (visited is monotone).
 * ------------------------------------------------------------------------- */
static int cmp_i32(const void *a, const void *b) {
  int32_t x = *(const int32_t *)a, y = *(const int32_t *)b;
  return (x > y) - (x < y);
}

typedef struct {
  int64_t n, *aptr, *deg, *cursor, nperm, odd_ptr, any_ptr;
  int32_t *adj, *score, *order;
  char *visited;
  int omega;
} trav_t;

/* any unvisited neighbour?  (advances the cursor past leading visited entries) */
static int has_unvisited(trav_t *t, int64_t v) {
  int64_t end = t->aptr[v] + t->deg[v];
  while (t->cursor[v] < end && t->visited[t->adj[t->cursor[v]]]) t->cursor[v]++;
  return t->cursor[v] < end;
}

/* visit(v): first appearance; maintain score[u] = |adj(u) ∩ W| for unvisited u */
static void visit(trav_t *t, int32_t v) {
  t->visited[v] = 1;
  t->order[t->nperm++] = v;
  for (int64_t k = t->aptr[v]; k < t->aptr[v] + t->deg[v]; ++k)
    if (!t->visited[t->adj[k]]) t->score[t->adj[k]]++;
  if (t->nperm > t->omega) {                 /* W drops its oldest entry */
    int32_t o = t->order[t->nperm - 1 - t->omega];
    for (int64_t k = t->aptr[o]; k < t->aptr[o] + t->deg[o]; ++k)
      if (!t->visited[t->adj[k]]) t->score[t->adj[k]]--;
  }
}

/* tier 3 / start: the unvisited node minimising (deg is even, id) */
static int32_t tier3(trav_t *t) {
  while (t->odd_ptr < t->n && (t->visited[t->odd_ptr] || t->deg[t->odd_ptr] % 2 == 0)) t->odd_ptr++;
  if (t->odd_ptr < t->n) return (int32_t)t->odd_ptr;
  while (t->any_ptr < t->n && t->visited[t->any_ptr]) t->any_ptr++;
  return (int32_t)t->any_ptr;
}

/* perm[n] (old id of new id r); P (appearances, capacity 2n, may be NULL);
 * stats[0]=|P|, stats[1]=jumps, stats[2]=window, stats[3]=cap. */
int ora_traverse(int64_t n, const int64_t *indptr, const int32_t *indices, int window, int cap,
                 int32_t *perm, int32_t *P, int64_t *stats) {
  const int64_t m = n > 0 ? indptr[n] : 0;
  int omega = window;
  if (omega <= 0) {
    omega = (int)(n > 0 ? (2 * m + n) / (2 * n) : 1);
    if (omega < 1) omega = 1;
    if (omega > 64) omega = 64;
  }
  const int K = cap > 0 ? cap : 32;
  trav_t t;
  memset(&t, 0, sizeof t);
  t.n = n; t.omega = omega;
  /* G_u: {i, j} for every edge j -> i, i != j; sorted; deduplicated */
  t.aptr = (int64_t *)calloc((size_t)n + 1, sizeof(int64_t));
  for (int64_t i = 0; i < n; ++i)
    for (int64_t k = indptr[i]; k < indptr[i + 1]; ++k)
      if (indices[k] != i) { t.aptr[i + 1]++; t.aptr[indices[k] + 1]++; }
  for (int64_t v = 0; v < n; ++v) t.aptr[v + 1] += t.aptr[v];
  t.adj = (int32_t *)malloc(sizeof(int32_t) * (size_t)(t.aptr[n] + 1));
  int64_t *fill = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n + 1));
  memcpy(fill, t.aptr, sizeof(int64_t) * (size_t)n);
  for (int64_t i = 0; i < n; ++i)
    for (int64_t k = indptr[i]; k < indptr[i + 1]; ++k)
      if (indices[k] != i) { t.adj[fill[i]++] = indices[k]; t.adj[fill[indices[k]]++] = (int32_t)i; }
  free(fill);
  t.deg = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n + 1));
  for (int64_t v = 0; v < n; ++v) {
    int64_t b = t.aptr[v], e = t.aptr[v + 1], w = b;
    qsort(t.adj + b, (size_t)(e - b), sizeof(int32_t), cmp_i32);
    for (int64_t k = b; k < e; ++k)
      if (k == b || t.adj[k] != t.adj[k - 1]) t.adj[w++] = t.adj[k];
    t.deg[v] = w - b;
  }
  t.visited = (char *)calloc((size_t)n + 1, 1);
  t.score = (int32_t *)calloc((size_t)n + 1, sizeof(int32_t));
  t.cursor = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n + 1));
  for (int64_t v = 0; v < n; ++v) t.cursor[v] = t.aptr[v];
  t.order = perm;
  int32_t *stk = (int32_t *)malloc(sizeof(int32_t) * (size_t)(2 * n + 2));
  int64_t sp = 0, plen = 0, t3 = 0;
  if (n > 0) {
    int32_t curr = tier3(&t); t3++;
    visit(&t, curr);
    if (P) P[plen] = curr;
    plen++;
    if (has_unvisited(&t, curr)) stk[sp++] = curr;
    while (t.nperm < n) {
      if (has_unvisited(&t, curr)) {                 /* tier 1: first K unvisited neighbours */
        int32_t best = -1;
        int taken = 0;
        for (int64_t k = t.cursor[curr]; k < t.aptr[curr] + t.deg[curr] && taken < K; ++k) {
          int32_t u = t.adj[k];
          if (t.visited[u]) continue;
          taken++;
          if (best < 0 || t.score[u] > t.score[best]) best = u;   /* ties -> smallest id */
        }
        curr = best;
        visit(&t, curr);
      } else {
        while (sp > 0 && !has_unvisited(&t, stk[sp - 1])) sp--;
        if (sp > 0) {
          curr = stk[--sp];                          /* tier 2: revisit */
        } else {
          curr = tier3(&t); t3++;                    /* tier 3: jump */
          visit(&t, curr);
        }
      }
      if (P) P[plen] = curr;
      plen++;
      if (has_unvisited(&t, curr)) stk[sp++] = curr;
    }
  }
  if (stats) { stats[0] = plen; stats[1] = t3 > 0 ? t3 - 1 : 0; stats[2] = omega; stats[3] = K; }
  free(t.aptr); free(t.adj); free(t.deg); free(t.visited); free(t.score); free(t.cursor); free(stk);
  return 0;
}

/* ---------------------------------------------------------------------------
 * L2 blocking (R24; oracle/blocks.py states the definition).  Plain:
 * G_u built as in ora_traverse; per visited node a full scan of the labels
 * present among its neighbours, counted with a scratch array.
 * label[n] out; stats[0] = sweeps run.  Returns 0.
 * ------------------------------------------------------------------------- */
static const int64_t *g_sort_deg;
static int cmp_deg_id(const void *a, const void *b) {
  int32_t x = *(const int32_t *)a, y = *(const int32_t *)b;
  if (g_sort_deg[x] != g_sort_deg[y]) return g_sort_deg[x] < g_sort_deg[y] ? -1 : 1;
  return (x > y) - (x < y);
}

int ora_l2_blocks(int64_t n, const int64_t *indptr, const int32_t *indices, int32_t B, int sweeps,
                  int32_t *label, int64_t *stats) {
  int64_t *aptr = (int64_t *)calloc((size_t)n + 1, sizeof(int64_t));
  for (int64_t i = 0; i < n; ++i)
    for (int64_t k = indptr[i]; k < indptr[i + 1]; ++k)
      if (indices[k] != i) { aptr[i + 1]++; aptr[indices[k] + 1]++; }
  for (int64_t v = 0; v < n; ++v) aptr[v + 1] += aptr[v];
  int32_t *adj = (int32_t *)malloc(sizeof(int32_t) * (size_t)(aptr[n] + 1));
  int64_t *fill = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n + 1));
  memcpy(fill, aptr, sizeof(int64_t) * (size_t)n);
  for (int64_t i = 0; i < n; ++i)
    for (int64_t k = indptr[i]; k < indptr[i + 1]; ++k)
      if (indices[k] != i) { adj[fill[i]++] = indices[k]; adj[fill[indices[k]]++] = (int32_t)i; }
  int64_t *deg = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n + 1));
  for (int64_t v = 0; v < n; ++v) {
    int64_t b = aptr[v], e = aptr[v + 1], w = b;
    qsort(adj + b, (size_t)(e - b), sizeof(int32_t), cmp_i32);
    for (int64_t k = b; k < e; ++k)
      if (k == b || adj[k] != adj[k - 1]) adj[w++] = adj[k];
    deg[v] = w - b;
  }
  int32_t *visit = (int32_t *)malloc(sizeof(int32_t) * (size_t)(n + 1));
  int64_t *size = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n + 1));
  int64_t *cnt = (int64_t *)calloc((size_t)n + 1, sizeof(int64_t));
  for (int64_t v = 0; v < n; ++v) { visit[v] = (int32_t)v; label[v] = (int32_t)v; size[v] = 1; }
  g_sort_deg = deg;
  qsort(visit, (size_t)n, sizeof(int32_t), cmp_deg_id);
  const int T = sweeps > 0 ? sweeps : 10;
  int run = 0;
  for (int it = 0; it < T; ++it) {
    run++;
    int64_t changed = 0;
    for (int64_t q = 0; q < n; ++q) {
      int32_t v = visit[q];
      if (deg[v] == 0) continue;
      for (int64_t k = aptr[v]; k < aptr[v] + deg[v]; ++k) cnt[label[adj[k]]]++;
      int32_t cur = label[v], best = cur;
      /* key (cnt, l == cur, -l), maximised; cur is always a candidate */
      for (int64_t k = aptr[v]; k < aptr[v] + deg[v]; ++k) {
        int32_t l = label[adj[k]];
        if (l == cur || size[l] >= B) continue;
        int better = cnt[l] > cnt[best] || (cnt[l] == cnt[best] && best != cur && l < best);
        if (better) best = l;
      }
      for (int64_t k = aptr[v]; k < aptr[v] + deg[v]; ++k) cnt[label[adj[k]]] = 0;
      if (best != cur) { size[cur]--; size[best]++; label[v] = best; changed++; }
    }
    if (changed * 1000 < n) break;
  }
  if (stats) stats[0] = run;
  free(aptr); free(adj); free(fill); free(deg); free(visit); free(size); free(cnt);
  return 0;
}
