/*
 * mega-synth v1 — seeded synthetic inputs shared by the oracle, the tests and
 * bench.py.  Test infrastructure: it holds NONE of the method's arithmetic
 * (no traversal, no attention); it only draws graphs and numbers.
 *
 * Graph model: a degree-corrected
 * stochastic block model with Chung–Lu power-law weights
 *     w_r = (r + r0)^(-1/(gamma-1)),  r = rank 0..n-1,
 * r0 chosen so the expected maximum in-degree m*w_0/sum(w) is ~d_cap; ranks are
 * assigned to node ids by a seeded random permutation (so input order carries
 * no locality) and every node gets a community uniform in [0, C).  Each draw t
 * picks a ~ w, then with probability mu b ~ w restricted to a's community,
 * else b ~ w, and emits (a -> b) (plus (b -> a) when undirected).  Duplicates
 * and self-loops are kept, so the edge count is exact.  Edge counts are
 * directed counts, Table II.
 *
 * RNG: counter-based splitmix64; element i of stream `seed` is
 * mix(seed + (i+1)*GOLDEN), i.e. the i-th output of a splitmix64 generator.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define GOLDEN 0x9E3779B97F4A7C15ULL

static inline uint64_t mix64(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}
static inline uint64_t draw(uint64_t seed, uint64_t i) { return mix64(seed + (i + 1) * GOLDEN); }
static inline double u01(uint64_t u) { return (double)(u >> 11) * (1.0 / 9007199254740992.0); }

uint64_t msynth_draw(uint64_t seed, uint64_t i) { return draw(seed, i); }

/* Vose alias table over weights w[0..k-1]. */
typedef struct { float *prob; int32_t *alias; } alias_t;

static void alias_build(const double *w, int64_t k, float *prob, int32_t *alias) {
  double sum = 0;
  for (int64_t i = 0; i < k; ++i) sum += w[i];
  double *q = (double *)malloc(sizeof(double) * (size_t)k);
  int64_t *small = (int64_t *)malloc(sizeof(int64_t) * (size_t)k);
  int64_t *large = (int64_t *)malloc(sizeof(int64_t) * (size_t)k);
  int64_t ns = 0, nl = 0;
  for (int64_t i = 0; i < k; ++i) {
    q[i] = w[i] * (double)k / sum;
    if (q[i] < 1.0) small[ns++] = i; else large[nl++] = i;
  }
  while (ns > 0 && nl > 0) {
    int64_t s = small[--ns], l = large[--nl];
    prob[s] = (float)q[s];
    alias[s] = (int32_t)l;
    q[l] = (q[l] + q[s]) - 1.0;
    if (q[l] < 1.0) small[ns++] = l; else large[nl++] = l;
  }
  while (nl > 0) { int64_t l = large[--nl]; prob[l] = 1.0f; alias[l] = (int32_t)l; }
  while (ns > 0) { int64_t s = small[--ns]; prob[s] = 1.0f; alias[s] = (int32_t)s; }
  free(q); free(small); free(large);
}

static inline int64_t alias_sample(const float *prob, const int32_t *alias, int64_t k, uint64_t u) {
  int64_t idx = (int64_t)(((u >> 32) * (uint64_t)k) >> 32);
  float coin = (float)(u & 0xffffffffULL) * (1.0f / 4294967296.0f);
  return coin < prob[idx] ? idx : alias[idx];
}

static double expected_max(double r0, double beta, int64_t n, double m) {
  double s = 0;
  for (int64_t r = 0; r < n; ++r) s += exp(-beta * log((double)r + r0));
  return m * exp(-beta * log(r0)) / s;
}

/*
 * Fills indptr[n+1] (int64, CSR by destination) and indices[m] (int32 source
 * ids), edges of each row in emission order.  stats[0] = duplicate edges,
 * stats[1] = self loops (informational).  Returns 0, or -1 on bad arguments.
 */
int msynth_graph(int64_t n, int64_t m, int directed, int32_t C, double mu, double gamma,
                 double d_cap, uint64_t seed, int64_t *indptr, int32_t *indices, int64_t *stats) {
  if (n <= 0 || m < 0 || n > 2147483647LL || m > 2147483647LL || C <= 0) return -1;
  if (!directed && (m & 1)) return -1;
  const double beta = 1.0 / (gamma - 1.0);
  /* r0: bisection in log space so that expected max degree ~ d_cap */
  double lo = 1e-3, hi = (double)n, r0 = 1.0;
  if (expected_max(lo, beta, n, (double)m) <= d_cap) r0 = lo;
  else {
    for (int it = 0; it < 40; ++it) {
      double mid = sqrt(lo * hi);
      if (expected_max(mid, beta, n, (double)m) > d_cap) lo = mid; else hi = mid;
    }
    r0 = sqrt(lo * hi);
  }
  const uint64_t s_perm = seed ^ 0x1111111111111111ULL, s_comm = seed ^ 0x2222222222222222ULL,
                 s_edge = seed ^ 0x3333333333333333ULL;
  /* rank -> node id via Fisher-Yates */
  int32_t *node_of_rank = (int32_t *)malloc(sizeof(int32_t) * (size_t)n);
  for (int64_t i = 0; i < n; ++i) node_of_rank[i] = (int32_t)i;
  for (int64_t i = n - 1; i > 0; --i) {
    int64_t j = (int64_t)((draw(s_perm, (uint64_t)i) >> 11) % (uint64_t)(i + 1));
    int32_t t = node_of_rank[i]; node_of_rank[i] = node_of_rank[j]; node_of_rank[j] = t;
  }
  double *w = (double *)malloc(sizeof(double) * (size_t)n);
  for (int64_t r = 0; r < n; ++r) w[node_of_rank[r]] = exp(-beta * log((double)r + r0));
  free(node_of_rank);
  int32_t *comm = (int32_t *)malloc(sizeof(int32_t) * (size_t)n);
  for (int64_t v = 0; v < n; ++v) comm[v] = (int32_t)(draw(s_comm, (uint64_t)v) % (uint64_t)C);
  /* global alias */
  float *gprob = (float *)malloc(sizeof(float) * (size_t)n);
  int32_t *galias = (int32_t *)malloc(sizeof(int32_t) * (size_t)n);
  alias_build(w, n, gprob, galias);
  /* per-community alias over members (members listed in id order) */
  int64_t *coff = (int64_t *)calloc((size_t)C + 1, sizeof(int64_t));
  for (int64_t v = 0; v < n; ++v) coff[comm[v] + 1]++;
  for (int32_t c = 0; c < C; ++c) coff[c + 1] += coff[c];
  int32_t *members = (int32_t *)malloc(sizeof(int32_t) * (size_t)n);
  int64_t *fill = (int64_t *)malloc(sizeof(int64_t) * (size_t)C);
  for (int32_t c = 0; c < C; ++c) fill[c] = coff[c];
  for (int64_t v = 0; v < n; ++v) members[fill[comm[v]]++] = (int32_t)v;
  free(fill);
  double *mw = (double *)malloc(sizeof(double) * (size_t)n);
  for (int64_t k = 0; k < n; ++k) mw[k] = w[members[k]];
  float *cprob = (float *)malloc(sizeof(float) * (size_t)n);
  int32_t *calias = (int32_t *)malloc(sizeof(int32_t) * (size_t)n);
  for (int32_t c = 0; c < C; ++c)
    if (coff[c + 1] > coff[c]) alias_build(mw + coff[c], coff[c + 1] - coff[c], cprob + coff[c], calias + coff[c]);
  free(mw); free(w);
  /* draws */
  const int64_t T = directed ? m : m / 2;
  int32_t *ea = (int32_t *)malloc(sizeof(int32_t) * (size_t)T);
  int32_t *eb = (int32_t *)malloc(sizeof(int32_t) * (size_t)T);
#pragma omp parallel for schedule(static)
  for (int64_t t = 0; t < T; ++t) {
    uint64_t h0 = draw(s_edge, 3 * (uint64_t)t), h1 = draw(s_edge, 3 * (uint64_t)t + 1),
             h2 = draw(s_edge, 3 * (uint64_t)t + 2);
    int64_t a = alias_sample(gprob, galias, n, h0);
    int64_t b;
    int32_t c = comm[a];
    if (u01(h1) < mu) {
      int64_t k = coff[c + 1] - coff[c];
      b = members[coff[c] + alias_sample(cprob + coff[c], calias + coff[c], k, h2)];
    } else {
      b = alias_sample(gprob, galias, n, h2);
    }
    ea[t] = (int32_t)a; eb[t] = (int32_t)b;
  }
  free(gprob); free(galias); free(cprob); free(calias); free(members); free(coff); free(comm);
  /* CSR by destination, stable in emission order: pair t emits (a->b) then (b->a) */
  memset(indptr, 0, sizeof(int64_t) * (size_t)(n + 1));
  for (int64_t t = 0; t < T; ++t) {
    indptr[eb[t] + 1]++;
    if (!directed) indptr[ea[t] + 1]++;
  }
  for (int64_t v = 0; v < n; ++v) indptr[v + 1] += indptr[v];
  int64_t *pos = (int64_t *)malloc(sizeof(int64_t) * (size_t)n);
  memcpy(pos, indptr, sizeof(int64_t) * (size_t)n);
  int64_t self_loops = 0;
  for (int64_t t = 0; t < T; ++t) {
    indices[pos[eb[t]]++] = ea[t];
    if (!directed) indices[pos[ea[t]]++] = eb[t];
    if (ea[t] == eb[t]) self_loops += directed ? 1 : 2;
  }
  free(pos); free(ea); free(eb);
  if (stats) {
    /* duplicates: per row, count repeated sources (hash-free: mark with a stamp array) */
    int64_t dups = 0;
    int64_t *stamp = (int64_t *)malloc(sizeof(int64_t) * (size_t)n);
    for (int64_t v = 0; v < n; ++v) stamp[v] = -1;
    for (int64_t v = 0; v < n; ++v)
      for (int64_t e = indptr[v]; e < indptr[v + 1]; ++e) {
        if (stamp[indices[e]] == v) dups++; else stamp[indices[e]] = v;
      }
    free(stamp);
    stats[0] = dups; stats[1] = self_loops;
  }
  return 0;
}

/* N(0, scale^2) via Box-Muller, element i from draw(seed, i). */
void msynth_normal_f32(uint64_t seed, int64_t count, float scale, float *out) {
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < count; ++i) {
    uint64_t u = draw(seed, (uint64_t)i);
    double u1 = ((double)(u >> 32) + 0.5) * (1.0 / 4294967296.0);
    double u2 = (double)(u & 0xffffffffULL) * (1.0 / 4294967296.0);
    out[i] = (float)(scale * sqrt(-2.0 * log(u1)) * cos(6.283185307179586 * u2));
  }
}

/* U[lo, hi), element i from draw(seed, i). */
void msynth_uniform_f32(uint64_t seed, int64_t count, float lo, float hi, float *out) {
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < count; ++i) out[i] = (float)(lo + (hi - lo) * u01(draw(seed, (uint64_t)i)));
}
