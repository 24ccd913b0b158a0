// NEXT-2: the paper's own representation — a path of node
// appearances with revisits, the graph stored as a band of width omega along it
// (Fig. 7) — built exactly (theta = 1: every edge
// covered) so GAT over it equals GAT over the input multiset (north_star).
//
// Traversal F (DESIGN.md R-band): R's tiers with coverage —
// every G_u edge starts uncovered; appending x to the path covers each
// uncovered {x, u} with u among the previous omega entries (owner (t, o));
// tier 1 = the first K neighbours of curr over uncovered edges (visited or
// not) by score |adj(v) ∩ last omega path entries|, ties to the smallest id;
// tier 2 = the stack (entries with uncovered edges), tier 3 = the unvisited
// node minimising (deg is even, id), then (R-band-1) a node with uncovered
// edges by the same key; stop when every node is visited and every edge
// covered.  Implemented independently of oracle/band.py; the band view is
// compared with it bit-exactly (tests/test_band_product.py).
//
// Per appearance t the device image holds: P[t]; lmask[t] bit o-1 = an in-edge
// of P[t] from P[t-o] through the pair (t, o); rmask[t] bit o-1 = an in-edge
// of P[t] from P[t+o] through (t+o, o); the multiplicities of those edges
// (uint16, lmask bits ascending then rmask bits) and of P[t]'s self-loops at
// its first appearance; the partial-state slot of appearances of nodes that
// appear more than once (merged per node in fixed order).
#include <algorithm>
#include <chrono>
#include <cstring>
#include <deque>
#include <new>

#include "mega_internal.h"

struct mega_band {
  int64_t n = 0, m = 0;
  int32_t omega = 0, cap = 0;
  std::vector<int32_t> P;          // appearances
  std::vector<uint64_t> own;       // own[t] bit o-1: G_u edge {P[t], P[t-o]} covered at t
  std::vector<uint64_t> lmask, rmask;
  std::vector<int32_t> cptr;       // [L+1] offsets into cnt
  std::vector<uint16_t> cnt;       // multiplicities (lmask bits, rmask bits), then self-loops
  std::vector<uint16_t> selfc;     // [L] self-loop count (first appearance only)
  std::vector<int32_t> slot;       // [L] partial slot or -1
  std::vector<int32_t> merges;     // [n_merge][3] (node, first slot, count)
  std::vector<int32_t> app_ptr;    // [n+1] appearances of each node (CSR over app_idx, appearance order)
  std::vector<int32_t> app_idx;    // [L]
  int32_t n_slots = 0;
  int64_t jumps = 0, virtual_edges = 0, edges_u = 0;
  double seconds = 0;
  // device image
  int device = -1;
  void *dev_base = nullptr;
  mega::BandDev dev;
};

namespace mega {
namespace {

constexpr int kBandArrays = 9;

struct G {
  std::vector<int64_t> beg;   // [n+1]
  std::vector<int32_t> nbr;   // sorted, unique
};

void build_gu(int64_t n, const int64_t *indptr, const int32_t *indices, G &g) {
  g.beg.assign(n + 1, 0);
  for (int64_t i = 0; i < n; ++i)
    for (int64_t e = indptr[i]; e < indptr[i + 1]; ++e)
      if (indices[e] != i) { g.beg[i + 1]++; g.beg[indices[e] + 1]++; }
  for (int64_t v = 0; v < n; ++v) g.beg[v + 1] += g.beg[v];
  std::vector<int32_t> tmp(g.beg[n]);
  std::vector<int64_t> fill(g.beg.begin(), g.beg.end() - 1);
  for (int64_t i = 0; i < n; ++i)
    for (int64_t e = indptr[i]; e < indptr[i + 1]; ++e) {
      const int32_t j = indices[e];
      if (j != i) { tmp[fill[i]++] = j; tmp[fill[j]++] = (int32_t)i; }
    }
  std::vector<int64_t> nb(n + 1, 0);
  for (int64_t v = 0; v < n; ++v) {
    int32_t *p = tmp.data() + g.beg[v], *q = tmp.data() + g.beg[v + 1];
    std::sort(p, q);
    nb[v + 1] = std::unique(p, q) - p;
  }
  for (int64_t v = 0; v < n; ++v) nb[v + 1] += nb[v];
  g.nbr.resize(nb[n]);
  for (int64_t v = 0; v < n; ++v) std::copy(tmp.data() + g.beg[v], tmp.data() + g.beg[v] + (nb[v + 1] - nb[v]),
                                            g.nbr.data() + nb[v]);
  g.beg.swap(nb);
}

// position of u in v's adjacency (must exist)
inline int64_t pos_of(const G &g, int32_t v, int32_t u) {
  const int32_t *p = g.nbr.data() + g.beg[v], *q = g.nbr.data() + g.beg[v + 1];
  const int32_t *r = std::lower_bound(p, q, u);
  return (r != q && *r == u) ? (r - g.nbr.data()) : -1;
}

mega_status traverse_f(int64_t n, const G &g, int omega, int K, mega_band &B) {
  std::vector<uint8_t> cov(g.nbr.size(), 0), visited(n, 0);
  std::vector<int64_t> head(g.beg.begin(), g.beg.end() - 1);   // entries before head are covered
  std::vector<int32_t> live(n), score(n, 0);
  for (int64_t v = 0; v < n; ++v) live[v] = (int32_t)(g.beg[v + 1] - g.beg[v]);
  const int64_t n_edges = (int64_t)g.nbr.size() / 2;
  int64_t covered = 0, n_visited = 0;
  B.edges_u = n_edges;
  std::vector<int32_t> stk;
  std::deque<int32_t> win;
  int64_t odd_u = 0, even_u = 0, odd_l = 0, even_l = 0;   // tier-3 cursors (ids ascending)
  auto deg = [&](int64_t v) { return g.beg[v + 1] - g.beg[v]; };
  auto append = [&](int32_t x) {
    const int64_t t = (int64_t)B.P.size();
    uint64_t own = 0;
    for (int o = 1; o <= omega && t - o >= 0; ++o) {
      const int32_t u = B.P[t - o];
      if (u == x) continue;
      const int64_t px = pos_of(g, x, u);
      if (px < 0 || cov[px]) continue;
      const int64_t pu = pos_of(g, u, x);
      cov[px] = cov[pu] = 1;
      --live[x];
      --live[u];
      ++covered;
      own |= 1ull << (o - 1);
    }
    B.P.push_back(x);
    B.own.push_back(own);
    if (!visited[x]) { visited[x] = 1; ++n_visited; }
    for (int64_t e = g.beg[x]; e < g.beg[x + 1]; ++e) ++score[g.nbr[e]];
    win.push_back(x);
    if ((int)win.size() > omega) {
      const int32_t w = win.front();
      win.pop_front();
      for (int64_t e = g.beg[w]; e < g.beg[w + 1]; ++e) --score[g.nbr[e]];
    }
  };
  auto tier3 = [&]() -> int32_t {
    if (n_visited < n) {
      while (odd_u < n && (visited[odd_u] || deg(odd_u) % 2 == 0)) ++odd_u;
      if (odd_u < n) return (int32_t)odd_u;
      while (even_u < n && (visited[even_u] || deg(even_u) % 2 != 0)) ++even_u;
      return (int32_t)even_u;
    }
    while (odd_l < n && (live[odd_l] == 0 || deg(odd_l) % 2 == 0)) ++odd_l;   // R-band-1
    if (odd_l < n) return (int32_t)odd_l;
    while (even_l < n && (live[even_l] == 0 || deg(even_l) % 2 != 0)) ++even_l;
    return even_l < n ? (int32_t)even_l : -1;
  };
  if (n == 0) return MEGA_OK;
  int32_t curr = tier3();
  append(curr);
  if (live[curr]) stk.push_back(curr);
  int32_t cand[64];
  while (n_visited < n || covered < n_edges) {
    // tier 1: the first K neighbours over uncovered edges, in id order
    int nc = 0;
    int64_t &h = head[curr];
    while (h < g.beg[curr + 1] && cov[h]) ++h;
    for (int64_t e = h; e < g.beg[curr + 1] && nc < K; ++e)
      if (!cov[e]) cand[nc++] = g.nbr[e];
    int32_t nxt;
    if (nc > 0) {
      nxt = cand[0];
      for (int c = 1; c < nc; ++c)
        if (score[cand[c]] > score[nxt]) nxt = cand[c];
    } else {
      while (!stk.empty() && live[stk.back()] == 0) stk.pop_back();
      if (!stk.empty()) {
        nxt = stk.back();            // tier 2: revisit
        stk.pop_back();
      } else {
        nxt = tier3();               // tier 3: jump
        if (nxt < 0) return fail(MEGA_ERR_STATE, "band traversal: no candidate with edges left uncovered");
        ++B.jumps;
      }
      if (pos_of(g, curr, nxt) < 0) ++B.virtual_edges;
    }
    curr = nxt;
    append(curr);
    if (live[curr]) stk.push_back(curr);
  }
  return MEGA_OK;
}

// directed multiplicities: rows of the input CSR sorted by source (a copy), counted by binary search
struct InCount {
  const int64_t *indptr;
  std::vector<int32_t> src;
  int32_t count(int32_t dst, int32_t s) const {
    auto p = src.begin() + indptr[dst], q = src.begin() + indptr[dst + 1];
    auto r = std::equal_range(p, q, s);
    return (int32_t)(r.second - r.first);
  }
};

mega_status band_arrays(int64_t n, const int64_t *indptr, const int32_t *indices, mega_band &B) {
  InCount ic{indptr, std::vector<int32_t>(indices, indices + indptr[n])};
  for (int64_t v = 0; v < n; ++v) std::sort(ic.src.begin() + indptr[v], ic.src.begin() + indptr[v + 1]);
  const int64_t L = (int64_t)B.P.size();
  const int omega = B.omega;
  B.lmask.assign(L, 0);
  B.rmask.assign(L, 0);
  B.selfc.assign(L, 0);
  std::vector<uint8_t> seen(n, 0);
  for (int64_t t = 0; t < L; ++t) {
    const int32_t x = B.P[t];
    if (!seen[x]) {
      seen[x] = 1;
      const int32_t s = ic.count(x, x);
      if (s > 65535) return fail(MEGA_ERR_UNSUPPORTED, "band layout: more than 65535 self-loops on a node");
      B.selfc[t] = (uint16_t)s;
    }
  }
  for (int64_t t = 0; t < L; ++t) {
    const int32_t x = B.P[t];
    for (int o = 1; o <= omega; ++o) {
      if (!((B.own[t] >> (o - 1)) & 1)) continue;
      const int32_t u = B.P[t - o];
      const int32_t cf = ic.count(x, u), cb = ic.count(u, x);   // u -> x, x -> u
      if (cf > 65535 || cb > 65535) return fail(MEGA_ERR_UNSUPPORTED, "band layout: an edge repeated more than 65535 times");
      if (cf) B.lmask[t] |= 1ull << (o - 1);
      if (cb) B.rmask[t - o] |= 1ull << (o - 1);
    }
  }
  B.cptr.assign(L + 1, 0);
  for (int64_t t = 0; t < L; ++t)
    B.cptr[t + 1] = B.cptr[t] + __builtin_popcountll(B.lmask[t]) + __builtin_popcountll(B.rmask[t]) + (B.selfc[t] ? 1 : 0);
  if ((int64_t)B.cptr[L] != B.cptr[L]) return fail(MEGA_ERR_UNSUPPORTED, "band layout too large");
  B.cnt.assign(B.cptr[L], 0);
  for (int64_t t = 0; t < L; ++t) {
    const int32_t x = B.P[t];
    int k = B.cptr[t];
    for (int o = 1; o <= omega; ++o)
      if ((B.lmask[t] >> (o - 1)) & 1) B.cnt[k++] = (uint16_t)ic.count(x, B.P[t - o]);
    for (int o = 1; o <= omega; ++o)
      if ((B.rmask[t] >> (o - 1)) & 1) B.cnt[k++] = (uint16_t)ic.count(x, B.P[t + o]);
    if (B.selfc[t]) B.cnt[k++] = B.selfc[t];
  }
  // partial slots: appearances of nodes that appear more than once, grouped by node (fixed order)
  std::vector<int32_t> napp(n, 0);
  for (int64_t t = 0; t < L; ++t) ++napp[B.P[t]];
  std::vector<int32_t> first_slot(n, -1);
  int32_t s = 0;
  for (int64_t v = 0; v < n; ++v)
    if (napp[v] > 1) {
      first_slot[v] = s;
      B.merges.insert(B.merges.end(), {(int32_t)v, s, napp[v]});
      s += napp[v];
    }
  B.n_slots = s;
  B.app_ptr.assign(n + 1, 0);
  for (int64_t v = 0; v < n; ++v) B.app_ptr[v + 1] = B.app_ptr[v] + napp[v];
  B.app_idx.assign(L, 0);
  {
    std::vector<int32_t> fill(B.app_ptr.begin(), B.app_ptr.end() - 1);
    for (int64_t t = 0; t < L; ++t) B.app_idx[fill[B.P[t]]++] = (int32_t)t;
  }
  B.slot.assign(L, -1);
  std::vector<int32_t> used(n, 0);
  for (int64_t t = 0; t < L; ++t) {
    const int32_t x = B.P[t];
    if (first_slot[x] >= 0) B.slot[t] = first_slot[x] + used[x]++;
  }
  return MEGA_OK;
}

size_t align256b(size_t x) { return (x + 255) / 256 * 256; }

size_t band_image(const mega_band &B, size_t offs[kBandArrays]) {
  const size_t L = B.P.size();
  const size_t sizes[kBandArrays] = {L * 4, L * 8, L * 8, (L + 1) * 4, B.cnt.size() * 2, L * 4, B.merges.size() * 4,
                                     B.app_ptr.size() * 4, L * 4};
  size_t off = 0;
  for (int i = 0; i < kBandArrays; ++i) {
    offs[i] = off;
    off = align256b(off + sizes[i]);
  }
  return off;
}

}  // namespace
}  // namespace mega

using namespace mega;

extern "C" {

mega_status mega_band_build(const mega_csr *csr, int32_t window, int32_t cap, mega_band **out) {
  clear_error();
  if (!csr || !out) return fail(MEGA_ERR_INVALID_ARGUMENT, "null argument");
  *out = nullptr;
  const int64_t n = csr->num_nodes, m = csr->num_edges;
  if (n <= 0 || n >= (1LL << 31) || m < 0 || m >= (1LL << 31)) return fail(MEGA_ERR_INVALID_GRAPH, "bad sizes");
  if (!csr->indptr || (m > 0 && !csr->indices)) return fail(MEGA_ERR_INVALID_ARGUMENT, "null CSR array");
  if (csr->indptr[0] != 0 || csr->indptr[n] != m) return fail(MEGA_ERR_INVALID_GRAPH, "indptr[0] != 0 or indptr[n] != m");
  for (int64_t i = 0; i < n; ++i)
    if (csr->indptr[i + 1] < csr->indptr[i]) return fail(MEGA_ERR_INVALID_GRAPH, "indptr not monotone");
  for (int64_t e = 0; e < m; ++e)
    if (csr->indices[e] < 0 || csr->indices[e] >= n) return fail(MEGA_ERR_INVALID_GRAPH, "source index out of range");
  if (window < 0 || window > 64 || cap < 0 || cap > 64)
    return fail(MEGA_ERR_INVALID_ARGUMENT, "window must be in [0, 64] and cap in [0, 64]");
  const auto t0 = std::chrono::steady_clock::now();
  mega_band *B = new (std::nothrow) mega_band();
  if (!B) return fail(MEGA_ERR_OUT_OF_MEMORY, "band allocation");
  try {
    B->n = n;
    B->m = m;
    B->omega = window > 0 ? window : (int32_t)std::min<int64_t>(64, std::max<int64_t>(1, (2 * m + n) / (2 * n)));
    B->cap = cap > 0 ? cap : 32;
    G g;
    build_gu(n, csr->indptr, csr->indices, g);
    mega_status s = traverse_f(n, g, B->omega, B->cap, *B);
    if (s == MEGA_OK) s = band_arrays(n, csr->indptr, csr->indices, *B);
    if (s != MEGA_OK) { delete B; return s; }
  } catch (const std::bad_alloc &) {
    delete B;
    return fail(MEGA_ERR_OUT_OF_MEMORY, "host allocation failed while building the band");
  }
  B->seconds = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
  *out = B;
  return MEGA_OK;
}

void mega_band_destroy(mega_band *B) { delete B; }

mega_status mega_band_view_get(const mega_band *B, mega_band_view *v) {
  clear_error();
  if (!B || !v) return fail(MEGA_ERR_INVALID_ARGUMENT, "null argument");
  std::memset(v, 0, sizeof *v);
  v->struct_size = sizeof *v;
  v->num_nodes = B->n;
  v->num_edges = B->m;
  v->length = (int64_t)B->P.size();
  v->window = B->omega;
  v->cap = B->cap;
  v->jumps = B->jumps;
  v->virtual_edges = B->virtual_edges;
  v->edges_u = B->edges_u;
  v->num_slots = B->n_slots;
  v->num_merges = (int64_t)B->merges.size() / 3;
  v->build_seconds = B->seconds;
  v->P = B->P.data();
  v->own = B->own.data();
  v->lmask = B->lmask.data();
  v->rmask = B->rmask.data();
  v->cptr = B->cptr.data();
  v->cnt = B->cnt.data();
  v->slot = B->slot.data();
  v->merges = B->merges.data();
  return MEGA_OK;
}

mega_status mega_band_device_bytes(const mega_band *B, size_t *bytes) {
  clear_error();
  if (!B || !bytes) return fail(MEGA_ERR_INVALID_ARGUMENT, "null argument");
  size_t offs[kBandArrays];
  *bytes = band_image(*B, offs);
  return MEGA_OK;
}

mega_status mega_band_bind_device(mega_band *B, void *dev_buf, size_t bytes, mega_stream_t stream) {
  clear_error();
  if (!B || !dev_buf) return fail(MEGA_ERR_INVALID_ARGUMENT, "null argument");
  if (reinterpret_cast<uintptr_t>(dev_buf) % 256) return fail(MEGA_ERR_INVALID_ARGUMENT, "dev_buf must be 256-byte aligned");
  size_t offs[kBandArrays];
  if (bytes < band_image(*B, offs)) return fail(MEGA_ERR_OUT_OF_MEMORY, "device buffer smaller than mega_band_device_bytes");
  int dev = 0;
  cudaError_t ce = cudaGetDevice(&dev);
  if (ce != cudaSuccess) return fail(MEGA_ERR_CUDA, std::string("cudaGetDevice: ") + cudaGetErrorString(ce));
  char *base = static_cast<char *>(dev_buf);
  const void *src[kBandArrays] = {B->P.data(), B->lmask.data(), B->rmask.data(), B->cptr.data(), B->cnt.data(),
                                  B->slot.data(), B->merges.data(), B->app_ptr.data(), B->app_idx.data()};
  const size_t L = B->P.size();
  const size_t sizes[kBandArrays] = {L * 4, L * 8, L * 8, (L + 1) * 4, B->cnt.size() * 2, L * 4, B->merges.size() * 4,
                                     B->app_ptr.size() * 4, L * 4};
  for (int i = 0; i < kBandArrays; ++i) {
    if (!sizes[i]) continue;
    ce = cudaMemcpyAsync(base + offs[i], src[i], sizes[i], cudaMemcpyHostToDevice, (cudaStream_t)stream);
    if (ce != cudaSuccess) return fail(MEGA_ERR_CUDA, std::string("band H2D copy: ") + cudaGetErrorString(ce));
  }
  B->device = dev;
  B->dev_base = dev_buf;
  BandDev &D = B->dev;
  D.P = reinterpret_cast<const int32_t *>(base + offs[0]);
  D.lmask = reinterpret_cast<const unsigned long long *>(base + offs[1]);
  D.rmask = reinterpret_cast<const unsigned long long *>(base + offs[2]);
  D.cptr = reinterpret_cast<const int32_t *>(base + offs[3]);
  D.cnt = reinterpret_cast<const uint16_t *>(base + offs[4]);
  D.slot = reinterpret_cast<const int32_t *>(base + offs[5]);
  D.merges = reinterpret_cast<const int32_t *>(base + offs[6]);
  D.app_ptr = reinterpret_cast<const int32_t *>(base + offs[7]);
  D.app_idx = reinterpret_cast<const int32_t *>(base + offs[8]);
  D.n_cnt = (int64_t)B->cnt.size();
  D.L = (int64_t)L;
  D.n = B->n;
  D.omega = B->omega;
  D.n_merges = (int32_t)(B->merges.size() / 3);
  D.n_slots = B->n_slots;
  return MEGA_OK;
}

}  // extern "C"

namespace mega {
const BandDev *band_dev(const mega_band *B, int &device) {
  device = B ? B->device : -1;
  return B && B->dev_base ? &B->dev : nullptr;
}
}  // namespace mega
