// a1. The MEGA reorganiser (host, once per graph) — mega_preprocess.
//
// PAPER.md §III-B (lines 186-235) and Algorithm 1 (lines 239-306): a single
// traversal derives a locality schedule; embeddings are then laid out in the
// order the traversal reaches them.  We keep MEGA's
// schedule but not its band-with-virtual-edges representation: the CSR is
// rewritten into an exact layout of our own, so the edge
// multiset is preserved (north_star).
//
// Traversal R (R8-R19; same reading as the oracle, implemented
// independently): G_u = symmetrised simple graph; score[u] = |adj(u) ∩ W| for
// the last omega first appearances W (Eq. (1)/(2)), kept
// incrementally in O(m); candidate tiers of PAPER.md:231-233 with the stack of
// PAPER.md:235.  Production cost O(m + K|P|): each adjacency list is compacted
// in place (order preserving) as visited entries are met, so every entry is
// dropped at most once.
#include <algorithm>
#include <chrono>
#include <functional>
#include <cstring>
#include <new>
#include <thread>

#include "mega_internal.h"

namespace mega {
namespace {

constexpr uint64_t kGolden = 0x9E3779B97F4A7C15ULL;
inline uint64_t splitmix(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}

template <typename F>
void parallel_for(int64_t n, F &&f) {
  unsigned hw = std::max(1u, std::min(32u, std::thread::hardware_concurrency()));
  if (n < 4096 || hw == 1) { f(0, n); return; }
  std::vector<std::thread> th;
  int64_t chunk = (n + hw - 1) / hw;
  for (unsigned t = 0; t < hw; ++t) {
    int64_t b = t * chunk, e = std::min(n, b + chunk);
    if (b >= e) break;
    th.emplace_back([&f, b, e] { f(b, e); });
  }
  for (auto &x : th) x.join();
}

// Undirected simple adjacency (traversal graph G_u), sorted ascending.
struct Adj {
  std::vector<int64_t> begin;  // [n+1] storage offsets
  std::vector<int64_t> head;   // live range [head[v], end[v])
  std::vector<int64_t> end;
  std::vector<int32_t> nbr;
};

void build_adj(int64_t n, const int64_t *indptr, const int32_t *indices, Adj &A) {
  A.begin.assign(n + 1, 0);
  for (int64_t i = 0; i < n; ++i)
    for (int64_t e = indptr[i]; e < indptr[i + 1]; ++e)
      if (indices[e] != i) { A.begin[i + 1]++; A.begin[indices[e] + 1]++; }
  for (int64_t v = 0; v < n; ++v) A.begin[v + 1] += A.begin[v];
  A.nbr.resize(A.begin[n]);
  std::vector<int64_t> fill(A.begin.begin(), A.begin.end() - 1);
  for (int64_t i = 0; i < n; ++i)
    for (int64_t e = indptr[i]; e < indptr[i + 1]; ++e) {
      int32_t j = indices[e];
      if (j != i) { A.nbr[fill[i]++] = j; A.nbr[fill[j]++] = (int32_t)i; }
    }
  A.head.resize(n);
  A.end.resize(n);
  parallel_for(n, [&](int64_t b, int64_t e) {
    for (int64_t v = b; v < e; ++v) {
      int32_t *p = A.nbr.data() + A.begin[v], *q = A.nbr.data() + A.begin[v + 1];
      std::sort(p, q);
      A.head[v] = A.begin[v];
      A.end[v] = A.begin[v] + (std::unique(p, q) - p);
    }
  });
}

struct Traversal {
  const int64_t n;
  const int omega, K;
  Adj &A;
  std::vector<uint8_t> visited;
  std::vector<int32_t> score;
  std::vector<int32_t> order;  // first appearances = perm
  int64_t odd_ptr = 0, any_ptr = 0;

  Traversal(int64_t n_, int omega_, int K_, Adj &A_) : n(n_), omega(omega_), K(K_), A(A_) {
    visited.assign(n, 0);
    score.assign(n, 0);
    order.reserve(n);
  }
  int64_t deg(int64_t v) const { return A.end[v] - A.begin[v]; }  // deg_u (before compaction)

  bool has_unvisited(int32_t v) {
    int64_t &h = A.head[v];
    const int64_t e = A.end[v];
    while (h < e && visited[A.nbr[h]]) ++h;
    return h < e;
  }
  void visit(int32_t v) {
    visited[v] = 1;
    order.push_back(v);
    for (int64_t k = A.head[v]; k < A.end[v]; ++k)
      if (!visited[A.nbr[k]]) score[A.nbr[k]]++;
    if ((int64_t)order.size() > omega) {  // the window drops its oldest first appearance
      int32_t o = order[order.size() - 1 - omega];
      for (int64_t k = A.head[o]; k < A.end[o]; ++k)
        if (!visited[A.nbr[k]]) score[A.nbr[k]]--;
    }
  }
  int32_t tier3() {  // min (deg_u is even, id) over unvisited nodes
    while (odd_ptr < n && (visited[odd_ptr] || (deg(odd_ptr) & 1) == 0)) ++odd_ptr;
    if (odd_ptr < n) return (int32_t)odd_ptr;
    while (any_ptr < n && visited[any_ptr]) ++any_ptr;
    return (int32_t)any_ptr;
  }
  // Tier 1: argmax score over the first K unvisited neighbours (ties -> first
  // = smallest id).  Compacts: the found candidates are moved next to the
  // unscanned tail and the skipped visited entries are dropped.
  int32_t tier1(int32_t v) {
    int32_t cand[64];
    int64_t r = A.head[v];
    const int64_t e = A.end[v];
    int found = 0;
    int32_t best = -1;
    while (r < e && found < K) {
      int32_t u = A.nbr[r++];
      if (visited[u]) continue;
      cand[found++] = u;
      if (best < 0 || score[u] > score[best]) best = u;
    }
    for (int i = 0; i < found; ++i) A.nbr[r - found + i] = cand[i];
    A.head[v] = r - found;
    return best;
  }

  void run(int64_t &path_len, int64_t &jumps) {
    std::vector<int32_t> stk;
    stk.reserve(1024);
    path_len = 0;
    int64_t t3 = 0;
    if (n == 0) { jumps = 0; return; }
    int32_t curr = tier3();
    ++t3;
    visit(curr);
    ++path_len;
    if (has_unvisited(curr)) stk.push_back(curr);
    while ((int64_t)order.size() < n) {
      if (has_unvisited(curr)) {
        curr = tier1(curr);
        visit(curr);
      } else {
        while (!stk.empty() && !has_unvisited(stk.back())) stk.pop_back();
        if (!stk.empty()) {
          curr = stk.back();  // tier 2: revisit
          stk.pop_back();
        } else {
          curr = tier3();     // tier 3: jump (virtual edge)
          ++t3;
          visit(curr);
        }
      }
      ++path_len;
      if (has_unvisited(curr)) stk.push_back(curr);
    }
    jumps = t3 - 1;
  }
};

// L2 blocking (R24; ours, not the paper's).  Size-constrained label
// propagation on G_u: nodes visited in ascending (deg_u, id); a node takes the
// label most frequent among its neighbours, preferring its own label on a tie,
// then the smallest label; a foreign label is eligible only while its block
// holds fewer than B nodes.  Sweeps stop at `max_sweeps` or once a sweep
// changes fewer than n/1000 labels.  Returns the label of every node.
std::vector<int32_t> l2_blocks(int64_t n, const Adj &A, int32_t B, int max_sweeps, int64_t &sweeps) {
  std::vector<int32_t> label(n), size(n, 1), visit(n), cnt(n, 0), seen;
  seen.reserve(1024);
  for (int64_t v = 0; v < n; ++v) label[v] = visit[v] = (int32_t)v;
  auto dg = [&](int32_t v) { return A.end[v] - A.begin[v]; };
  std::stable_sort(visit.begin(), visit.end(), [&](int32_t a, int32_t b) { return dg(a) < dg(b); });
  sweeps = 0;
  for (int it = 0; it < max_sweeps; ++it) {
    ++sweeps;
    int64_t changed = 0;
    for (int32_t v : visit) {
      if (dg(v) == 0) continue;
      seen.clear();
      for (int64_t k = A.begin[v]; k < A.end[v]; ++k) {
        int32_t l = label[A.nbr[k]];
        if (cnt[l]++ == 0) seen.push_back(l);
      }
      const int32_t cur = label[v];
      int32_t best = cur, bc = cnt[cur];
      for (int32_t l : seen) {
        if (l == cur || size[l] >= B) continue;
        if (cnt[l] > bc || (cnt[l] == bc && best != cur && l < best)) { best = l; bc = cnt[l]; }
      }
      for (int32_t l : seen) cnt[l] = 0;
      if (best != cur) { label[v] = best; --size[cur]; ++size[best]; ++changed; }
    }
    if (changed * 1000 < n) break;
  }
  return label;
}

void items_for(const std::vector<int32_t> &ptr, int32_t S, std::vector<int32_t> &items,
               std::vector<int32_t> &splits, int32_t &nslots) {
  const int64_t rows = (int64_t)ptr.size() - 1;
  items.clear();
  splits.clear();
  items.reserve(rows * 4);
  int32_t slot = 0;
  for (int64_t r = 0; r < rows; ++r) {
    int32_t b = ptr[r], e = ptr[r + 1];
    if (e - b <= S) {
      items.insert(items.end(), {(int32_t)r, b, e, -1});
    } else {
      int32_t nseg = (e - b + S - 1) / S;
      splits.insert(splits.end(), {(int32_t)r, slot, nseg});
      for (int32_t k = 0; k < nseg; ++k)
        items.insert(items.end(), {(int32_t)r, b + k * S, std::min(e, b + (k + 1) * S), slot + k});
      slot += nseg;
    }
  }
  nslots = slot;
}

}  // namespace

void compute_class_histograms(Part &P, int64_t n) {
  for (int c = 0; c < 64; ++c) P.out_cls[c] = P.in_cls[c] = 0;
  for (int64_t v = 0; v < n; ++v) P.out_cls[degree_class(P.cindptr[v + 1] - P.cindptr[v])]++;
  for (size_t r = 0; r + 1 < P.indptr.size(); ++r) P.in_cls[degree_class(P.indptr[r + 1] - P.indptr[r])]++;
}

mega_status build_layout(const mega_csr *csr, const mega_schedule_opts *opts, mega_layout *L) {
  auto t0 = std::chrono::steady_clock::now();
  const int64_t n = csr->num_nodes, m = csr->num_edges;
  const int64_t *indptr = csr->indptr;
  const int32_t *indices = csr->indices;
  L->n = n;
  L->m = m;
  L->opts = *opts;
  const int k = opts->num_parts;
  int omega = opts->window;
  if (omega <= 0) omega = (int)std::min<int64_t>(64, std::max<int64_t>(1, (2 * m + n) / (2 * n)));
  const int K = opts->candidate_cap > 0 ? opts->candidate_cap : 32;
  // S: work-item segment size.  Items are taken with a static grid stride, so the kernel ends
  // with the warp whose items sum to the most edges; 256 keeps that within ~13% of the mean on
  // products and reddit (measured best: products 81.1 ms/step at 256 vs 85.6 at round 1's
  // m/(148*256) = 1664; reddit 16.7 vs 21.4 at 3040)
  int32_t S = opts->seg_edges;
  if (S <= 0) S = 256;

  // ---- node order ----
  int64_t path_len = n, jumps = 0, sweeps = 0, nblocks = n;
  L->perm.resize(n);
  Adj A;
  std::vector<int32_t> label;
  if (opts->block_rows > 0 || opts->order == MEGA_ORDER_TRAVERSAL) build_adj(n, indptr, indices, A);
  if (opts->block_rows > 0)  // before the traversal compacts the adjacency lists
    label = l2_blocks(n, A, opts->block_rows, opts->block_sweeps > 0 ? opts->block_sweeps : 10, sweeps);
  switch (opts->order) {
    case MEGA_ORDER_TRAVERSAL: {
      Traversal T(n, omega, K, A);
      T.run(path_len, jumps);
      L->perm = std::move(T.order);
      break;
    }
    case MEGA_ORDER_IDENTITY:
      for (int64_t i = 0; i < n; ++i) L->perm[i] = (int32_t)i;
      break;
    case MEGA_ORDER_DEGREE: {
      for (int64_t i = 0; i < n; ++i) L->perm[i] = (int32_t)i;
      std::stable_sort(L->perm.begin(), L->perm.end(), [&](int32_t a, int32_t b) {
        return indptr[a + 1] - indptr[a] > indptr[b + 1] - indptr[b];
      });
      break;
    }
    case MEGA_ORDER_RANDOM: {
      for (int64_t i = 0; i < n; ++i) L->perm[i] = (int32_t)i;
      for (int64_t i = n - 1, kk = 0; i > 0; --i, ++kk) {
        uint64_t u = splitmix(opts->seed + (uint64_t)(kk + 1) * kGolden);
        int64_t j = (int64_t)((u >> 11) % (uint64_t)(i + 1));
        std::swap(L->perm[i], L->perm[j]);
      }
      break;
    }
    default:
      return fail(MEGA_ERR_INVALID_ARGUMENT, "unknown order");
  }
  if (opts->block_rows > 0) {  // stable regroup by block, blocks ranked by first position
    std::vector<int32_t> rank(n, -1), start;
    nblocks = 0;
    for (int64_t r = 0; r < n; ++r) {
      int32_t &k = rank[label[L->perm[r]]];
      if (k < 0) { k = (int32_t)nblocks++; start.push_back(0); }
      start[k]++;
    }
    int32_t acc = 0;
    for (auto &c : start) { int32_t t = c; c = acc; acc += t; }
    std::vector<int32_t> grouped(n);
    for (int64_t r = 0; r < n; ++r) grouped[start[rank[label[L->perm[r]]]]++] = L->perm[r];
    L->perm.swap(grouped);
  }
  { std::vector<int32_t>().swap(A.nbr); std::vector<int64_t>().swap(A.begin); }
  L->new_of_old.resize(n);
  for (int64_t r = 0; r < n; ++r) L->new_of_old[L->perm[r]] = (int32_t)r;

  // ---- (i) relabelled CSR: rows sorted by (new src, original position) ----
  std::vector<int32_t> ip(n + 1), src(m), eid(m);
  ip[0] = 0;
  for (int64_t r = 0; r < n; ++r) {
    int64_t o = L->perm[r];
    ip[r + 1] = ip[r] + (int32_t)(indptr[o + 1] - indptr[o]);
  }
  const int32_t *nofo = L->new_of_old.data();
  parallel_for(n, [&](int64_t b, int64_t e) {
    std::vector<uint64_t> keys;
    for (int64_t r = b; r < e; ++r) {
      int64_t o = L->perm[r], e0 = indptr[o], e1 = indptr[o + 1];
      keys.resize(e1 - e0);
      for (int64_t q = e0; q < e1; ++q) keys[q - e0] = ((uint64_t)(uint32_t)nofo[indices[q]] << 32) | (uint32_t)q;
      std::sort(keys.begin(), keys.end());
      int64_t base = ip[r];
      for (size_t q = 0; q < keys.size(); ++q) {
        src[base + q] = (int32_t)(keys[q] >> 32);
        eid[base + q] = (int32_t)(keys[q] & 0xffffffffu);
      }
    }
  });

  // ---- (iv) partitions: b_p = min{r : ip[r] >= ceil(p m / k)} ----
  L->bounds.assign(k + 1, 0);
  for (int p = 1; p < k; ++p) {
    int64_t t = (p * m + k - 1) / k;
    L->bounds[p] = (int32_t)(std::lower_bound(ip.begin(), ip.end(), (int32_t)t) - ip.begin());
  }
  L->bounds[k] = (int32_t)n;

  // ---- per part: (ii) CSC, (iii) work items ----
  L->parts.resize(k);
  int64_t max_out = 0;
  for (int p = 0; p < k; ++p) {
    Part &P = L->parts[p];
    P.row_begin = L->bounds[p];
    P.row_end = L->bounds[p + 1];
    const int64_t rows = P.row_end - P.row_begin, e0 = ip[P.row_begin], e1 = ip[P.row_end], E = e1 - e0;
    P.indptr.resize(rows + 1);
    for (int64_t r = 0; r <= rows; ++r) P.indptr[r] = (int32_t)(ip[P.row_begin + r] - e0);
    P.src.assign(src.begin() + e0, src.begin() + e1);
    P.eid.assign(eid.begin() + e0, eid.begin() + e1);
    P.cindptr.assign(n + 1, 0);
    for (int64_t q = 0; q < E; ++q) P.cindptr[P.src[q] + 1]++;
    for (int64_t v = 0; v < n; ++v) {
      max_out = std::max<int64_t>(max_out, P.cindptr[v + 1]);
      P.cindptr[v + 1] += P.cindptr[v];
    }
    P.cdst.resize(E);
    P.cpos.resize(E);
    P.csr2csc.resize(E);
    std::vector<int32_t> fill(P.cindptr.begin(), P.cindptr.end() - 1);
    for (int64_t r = 0; r < rows; ++r)
      for (int32_t q = P.indptr[r]; q < P.indptr[r + 1]; ++q) {
        int32_t c = fill[P.src[q]]++;
        P.cdst[c] = (int32_t)r;
        P.cpos[c] = q;
        P.csr2csc[q] = c;
      }
    compute_class_histograms(P, n);
    items_for(P.indptr, S, P.fwd_items, P.fwd_splits, P.n_fwd_slots);
    items_for(P.cindptr, S, P.bwd_items, P.bwd_splits, P.n_bwd_slots);
  }

  // ---- statistics ----
  mega_layout_stats &st = L->stats;
  std::memset(&st, 0, sizeof st);
  st.struct_size = sizeof st;
  st.num_nodes = n;
  st.num_edges = m;
  st.num_parts = k;
  st.window = omega;
  st.candidate_cap = K;
  st.seg_edges = S;
  st.order = opts->order;
  st.path_length = path_len;
  st.revisits = path_len - n;
  st.jumps = jumps;
  int64_t max_in = 0;
  for (int64_t r = 0; r < n; ++r) max_in = std::max<int64_t>(max_in, ip[r + 1] - ip[r]);
  st.max_in_degree = max_in;
  {  // out-degree over the whole graph
    std::vector<int64_t> od(n, 0);
    for (int64_t q = 0; q < m; ++q) od[src[q]]++;
    int64_t mo = 0;
    for (int64_t v = 0; v < n; ++v) mo = std::max(mo, od[v]);
    st.max_out_degree = mo;
  }
  (void)max_out;
  {  // sum over 64-row tiles of distinct sources
    std::vector<int32_t> stamp(n, -1);
    int64_t tot = 0;
    for (int64_t t = 0; t < n; t += 64) {
      int32_t tile = (int32_t)(t / 64);
      for (int64_t q = ip[t]; q < ip[std::min(n, t + 64)]; ++q)
        if (stamp[src[q]] != tile) { stamp[src[q]] = tile; ++tot; }
    }
    st.tile_unique_sources = tot;
  }
  st.block_rows = opts->block_rows;
  st.num_blocks = opts->block_rows > 0 ? nblocks : 0;
  st.block_sweeps = sweeps;
  st.preprocess_seconds = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
  return MEGA_OK;
}

}  // namespace mega
