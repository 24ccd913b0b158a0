// C ABI: errors, options, layout lifetime, views, persistence and device binding.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <functional>
#include <cstdlib>
#include <cstring>
#include <new>

#include "mega_internal.h"

namespace mega {
static thread_local std::string g_last_error;

mega_status fail(mega_status s, const std::string &msg) {
  g_last_error = msg;
  return s;
}
void clear_error() { g_last_error.clear(); }

static const size_t kAlign = 256;
static size_t align_up(size_t x) { return (x + kAlign - 1) / kAlign * kAlign; }

// Device image of one part: kImageArrays int32 arrays at 256-byte aligned offsets (the view
// arrays, the chunk schedules, the k-GPU item lists and halo plan, the destination-pass order).
std::vector<int32_t> make_chunks(const std::vector<int32_t> &items, int q, int cap) {
  std::vector<int32_t> c;
  const int64_t n = (int64_t)items.size() / 4;
  if (n < kChunkMinItems) q = 0;   // small graphs: every item its own chunk (parallelism over latency)
  c.reserve(n / 4 + 2);
  c.push_back(0);
  int64_t cost = 0, cnt = 0;
  for (int64_t i = 0; i < n; ++i) {
    cost += (int64_t)items[4 * i + 2] - items[4 * i + 1] + kChunkItemCost;
    if (++cnt >= cap || cost >= q) {
      c.push_back((int32_t)(i + 1));
      cost = cnt = 0;
    }
  }
  if (c.back() != (int32_t)n) c.push_back((int32_t)n);
  return c;
}

int chunk_quantum(bool fwd) {
  const char *e = std::getenv(fwd ? "MEGA_SCHED_Q" : "MEGA_SCHED_QB");
  return e ? std::max(0, std::atoi(e)) : (fwd ? kChunkEdgesFwd : kChunkEdgesBwd);
}

// Forward work split by source owner for the k-GPU path:
// part p's row r has its edges sorted by new source id, so the edges from p's own
// rows [b_p, b_{p+1}) (block (p,p), computable before any exchange) are one
// contiguous range [l0, l1) and the remote ones are [e0, l0) and [l1, e1).
// Each range is cut into segments of <= S edges.  A row whose edges form a single
// segment is finalised by the pass that owns it (slot -1); every other row gets a
// contiguous block of slots (local segments first) and a split record
// (row, first_slot, nseg) for the fixed-order merge after the remote pass.  Rows
// without edges are finalised (out = 0, lse = -inf) by the local pass.
void dist_items(const mega_layout *L, int part, std::vector<int32_t> &local, std::vector<int32_t> &remote,
                std::vector<int32_t> &splits, int32_t &nslots) {
  const Part &P = L->parts[part];
  const int32_t b0 = L->bounds[part], b1 = L->bounds[part + 1];
  const int32_t S = (int32_t)std::max<int64_t>(1, L->stats.seg_edges);
  local.clear(); remote.clear(); splits.clear();
  nslots = 0;
  const int64_t rows = (int64_t)P.indptr.size() - 1;
  for (int64_t r = 0; r < rows; ++r) {
    const int32_t e0 = P.indptr[r], e1 = P.indptr[r + 1];
    if (e1 == e0) { local.insert(local.end(), {(int32_t)r, e0, e0, -1}); continue; }
    const int32_t *sb = P.src.data() + e0, *se = P.src.data() + e1;
    const int32_t l0 = e0 + (int32_t)(std::lower_bound(sb, se, b0) - sb);
    const int32_t l1 = e0 + (int32_t)(std::lower_bound(sb, se, b1) - sb);
    const int32_t rng[3][3] = {{l0, l1, 1}, {e0, l0, 0}, {l1, e1, 0}};   // (begin, end, is_local)
    int32_t nseg = 0;
    for (auto &q : rng) if (q[1] > q[0]) nseg += (q[1] - q[0] + S - 1) / S;
    const bool single = nseg == 1;
    const int32_t base = single ? -1 : nslots;
    int32_t k = 0;
    for (auto &q : rng)
      for (int32_t b = q[0]; b < q[1]; b += S) {
        std::vector<int32_t> &dst = q[2] ? local : remote;
        dst.insert(dst.end(), {(int32_t)r, b, std::min(q[1], b + S), single ? -1 : base + k});
        ++k;
      }
    if (!single) {
      splits.insert(splits.end(), {(int32_t)r, base, nseg});
      nslots += nseg;
    }
  }
}

// NEXT-1: exchange only the rows a peer's edges reference.  Part p's
// CSC row j is non-empty exactly when some in-edge of p's rows comes from source j, so
// p needs from q the rows j in [b_q, b_{q+1}) with a non-empty CSC row in part p, and
// sends to q its own rows with a non-empty CSC row in part q.  The same lists, read the
// other way, route the backward's partial [dWh | der] rows back to their owners.
void halo_plan(const mega_layout *L, int part, std::vector<int32_t> &send_idx, std::vector<int32_t> &send_off,
               std::vector<int32_t> &recv_idx, std::vector<int32_t> &recv_off, std::vector<int32_t> &pos) {
  const int k = (int)L->parts.size();
  const Part &P = L->parts[part];
  const int32_t b0 = L->bounds[part], b1 = L->bounds[part + 1], rows = b1 - b0;
  send_idx.clear(); recv_idx.clear();
  send_off.assign(k + 1, 0);
  recv_off.assign(k + 1, 0);
  pos.assign((size_t)std::max(0, k - 1) * rows, -1);
  int slot = 0;
  for (int q = 0; q < k; ++q) {
    send_off[q] = (int32_t)send_idx.size();
    recv_off[q] = (int32_t)recv_idx.size();
    if (q == part) continue;
    const Part &Q = L->parts[q];
    for (int32_t j = b0; j < b1; ++j)   // own rows that q's edges reference
      if (Q.cindptr[j + 1] > Q.cindptr[j]) send_idx.push_back(j);
    for (int32_t j = L->bounds[q]; j < L->bounds[q + 1]; ++j)   // q's rows that this part's edges reference
      if (P.cindptr[j + 1] > P.cindptr[j]) recv_idx.push_back(j);
    // where q's partial of own row j lands in the receive buffer (q packs its partials of this
    // part's rows in the order of this list, the buffer holds the peers' blocks in peer order)
    for (int32_t t = send_off[q]; t < (int32_t)send_idx.size(); ++t)
      pos[(size_t)slot * rows + (send_idx[t] - b0)] = t;
    ++slot;
  }
  send_off[k] = (int32_t)send_idx.size();
  recv_off[k] = (int32_t)recv_idx.size();
}

size_t part_image_bytes(const mega_layout *L, int part, size_t offs[kImageArrays]) {
  const Part &P = L->parts[part];
  std::vector<int32_t> dl, dr, ds, hs, hso, hr, hro, hp;
  int32_t nsl = 0;
  if (L->parts.size() > 1) {
    dist_items(L, part, dl, dr, ds, nsl);
    halo_plan(L, part, hs, hso, hr, hro, hp);
  }
  const size_t sizes[kImageArrays] = {P.indptr.size(), P.src.size(), P.cindptr.size(), P.cdst.size(),
                                      P.csr2csc.size(), P.fwd_items.size(), P.fwd_splits.size(),
                                      P.bwd_items.size(), P.bwd_splits.size(),
                                      make_chunks(P.fwd_items, chunk_quantum(true), kChunkCapFwd).size(),
                                      make_chunks(P.bwd_items, chunk_quantum(false), kChunkCapBwd).size(), 0, 0,
                                      P.cpos.size(),
                                      dl.size(), dr.size(), ds.size(), hs.size(), hr.size(), hp.size(),
                                      P.indptr.size() - 1};
  size_t off = 0;
  for (int i = 0; i < kImageArrays; ++i) {
    offs[i] = off;
    off = align_up(off + sizes[i] * sizeof(int32_t));
  }
  return off;
}
}  // namespace mega

using namespace mega;

extern "C" {

int mega_abi_version(void) { return MEGA_ABI_VERSION; }

const char *mega_status_string(mega_status s) {
  switch (s) {
    case MEGA_OK: return "MEGA_OK";
    case MEGA_ERR_INVALID_ARGUMENT: return "MEGA_ERR_INVALID_ARGUMENT";
    case MEGA_ERR_INVALID_GRAPH: return "MEGA_ERR_INVALID_GRAPH";
    case MEGA_ERR_UNSUPPORTED: return "MEGA_ERR_UNSUPPORTED";
    case MEGA_ERR_OUT_OF_MEMORY: return "MEGA_ERR_OUT_OF_MEMORY";
    case MEGA_ERR_CUDA: return "MEGA_ERR_CUDA";
    case MEGA_ERR_STATE: return "MEGA_ERR_STATE";
    case MEGA_ERR_IO: return "MEGA_ERR_IO";
    case MEGA_ERR_NCCL: return "MEGA_ERR_NCCL";
  }
  return "MEGA_ERR_UNKNOWN";
}

const char *mega_last_error(void) { return g_last_error.c_str(); }

void mega_schedule_opts_init(mega_schedule_opts *o) {
  if (!o) return;
  std::memset(o, 0, sizeof *o);
  o->struct_size = sizeof *o;
  o->order = MEGA_ORDER_TRAVERSAL;
  o->num_parts = 1;
}

mega_status mega_preprocess(const mega_csr *csr, const mega_schedule_opts *opts, mega_layout **out) {
  clear_error();
  if (!csr || !opts || !out) return fail(MEGA_ERR_INVALID_ARGUMENT, "null argument");
  *out = nullptr;
  if (opts->struct_size != sizeof(mega_schedule_opts))
    return fail(MEGA_ERR_INVALID_ARGUMENT, "mega_schedule_opts.struct_size mismatch (call mega_schedule_opts_init)");
  const int64_t n = csr->num_nodes, m = csr->num_edges;
  if (n <= 0 || n >= (1LL << 31)) return fail(MEGA_ERR_INVALID_GRAPH, "num_nodes must be in [1, 2^31)");
  if (m < 0 || m >= (1LL << 31)) return fail(MEGA_ERR_INVALID_GRAPH, "num_edges must be in [0, 2^31)");
  if (!csr->indptr || (m > 0 && !csr->indices)) return fail(MEGA_ERR_INVALID_ARGUMENT, "null CSR array");
  if (opts->num_parts < 1 || opts->num_parts > 1024) return fail(MEGA_ERR_INVALID_ARGUMENT, "num_parts must be in [1, 1024]");
  if (opts->candidate_cap < 0 || opts->candidate_cap > 64)
    return fail(MEGA_ERR_INVALID_ARGUMENT, "candidate_cap must be in [0, 64]");
  if (opts->window < 0 || opts->seg_edges < 0) return fail(MEGA_ERR_INVALID_ARGUMENT, "negative window/seg_edges");
  if (opts->block_rows < 0 || opts->block_sweeps < 0 || opts->block_sweeps > 1000)
    return fail(MEGA_ERR_INVALID_ARGUMENT, "block_rows must be >= 0 and block_sweeps in [0, 1000]");
  if (opts->order < 0 || opts->order > MEGA_ORDER_RANDOM) return fail(MEGA_ERR_INVALID_ARGUMENT, "unknown order");
  if (csr->indptr[0] != 0 || csr->indptr[n] != m) return fail(MEGA_ERR_INVALID_GRAPH, "indptr[0] != 0 or indptr[n] != m");
  for (int64_t i = 0; i < n; ++i)
    if (csr->indptr[i + 1] < csr->indptr[i]) return fail(MEGA_ERR_INVALID_GRAPH, "indptr not monotone");
  for (int64_t e = 0; e < m; ++e)
    if (csr->indices[e] < 0 || csr->indices[e] >= n)
      return fail(MEGA_ERR_INVALID_GRAPH, "source index out of range at edge " + std::to_string(e));
  mega_layout *L = new (std::nothrow) mega_layout();
  if (!L) return fail(MEGA_ERR_OUT_OF_MEMORY, "layout allocation");
  try {
    mega_status s = build_layout(csr, opts, L);
    if (s != MEGA_OK) { delete L; return s; }
  } catch (const std::bad_alloc &) {
    delete L;
    return fail(MEGA_ERR_OUT_OF_MEMORY, "host allocation failed while building the layout");
  }
  *out = L;
  return MEGA_OK;
}

void mega_layout_destroy(mega_layout *L) { delete L; }

mega_status mega_layout_stats_get(const mega_layout *L, mega_layout_stats *out) {
  clear_error();
  if (!L || !out) return fail(MEGA_ERR_INVALID_ARGUMENT, "null argument");
  *out = L->stats;
  return MEGA_OK;
}

mega_status mega_layout_view_get(const mega_layout *L, int32_t part, mega_layout_view *v) {
  clear_error();
  if (!L || !v) return fail(MEGA_ERR_INVALID_ARGUMENT, "null argument");
  if (part < 0 || part >= (int32_t)L->parts.size()) return fail(MEGA_ERR_INVALID_ARGUMENT, "part out of range");
  const Part &P = L->parts[part];
  std::memset(v, 0, sizeof *v);
  v->struct_size = sizeof *v;
  v->num_nodes = L->n;
  v->num_edges = L->m;
  v->row_begin = P.row_begin;
  v->row_end = P.row_end;
  v->part_edges = (int64_t)P.src.size();
  v->num_fwd_items = (int64_t)P.fwd_items.size() / 4;
  v->num_fwd_splits = (int64_t)P.fwd_splits.size() / 3;
  v->num_bwd_items = (int64_t)P.bwd_items.size() / 4;
  v->num_bwd_splits = (int64_t)P.bwd_splits.size() / 3;
  v->num_parts = (int64_t)L->parts.size();
  v->perm = L->perm.data();
  v->new_of_old = L->new_of_old.data();
  v->bounds = L->bounds.data();
  v->indptr = P.indptr.data();
  v->src = P.src.data();
  v->eid = P.eid.data();
  v->cindptr = P.cindptr.data();
  v->cdst = P.cdst.data();
  v->cpos = P.cpos.data();
  v->csr2csc = P.csr2csc.data();
  v->fwd_items = P.fwd_items.data();
  v->fwd_splits = P.fwd_splits.data();
  v->bwd_items = P.bwd_items.data();
  v->bwd_splits = P.bwd_splits.data();
  return MEGA_OK;
}

mega_status mega_layout_dist_view_get(mega_layout *L, int32_t part, mega_layout_dist_view *v) {
  clear_error();
  if (!L || !v) return fail(MEGA_ERR_INVALID_ARGUMENT, "null argument");
  if (part < 0 || part >= (int32_t)L->parts.size()) return fail(MEGA_ERR_INVALID_ARGUMENT, "part out of range");
  Part &P = L->parts[part];
  std::memset(v, 0, sizeof *v);
  v->struct_size = sizeof *v;
  if (L->parts.size() > 1) {
    dist_items(L, part, P.dl_items, P.dr_items, P.d_splits, P.n_d_slots);
    halo_plan(L, part, P.hsend_idx, P.hsend_off, P.hrecv_idx, P.hrecv_off, P.hpos);
    v->num_send = (int64_t)P.hsend_idx.size();
    v->num_recv = (int64_t)P.hrecv_idx.size();
    v->full_recv_rows = L->n - (P.row_end - P.row_begin);
    v->send_idx = P.hsend_idx.data();
    v->send_off = P.hsend_off.data();
    v->recv_idx = P.hrecv_idx.data();
    v->recv_off = P.hrecv_off.data();
    auto first_ge = [](const std::vector<int32_t> &a, int stride, int32_t x) {
      int64_t lo = 0, hi = (int64_t)a.size() / stride;
      while (lo < hi) { int64_t mid = (lo + hi) / 2; if (a[mid * stride] < x) lo = mid + 1; else hi = mid; }
      return lo;
    };
    v->bwd_own_items_begin = first_ge(P.bwd_items, 4, (int32_t)P.row_begin);
    v->bwd_own_items_end = first_ge(P.bwd_items, 4, (int32_t)P.row_end);
    v->bwd_own_splits_begin = first_ge(P.bwd_splits, 3, (int32_t)P.row_begin);
    v->bwd_own_splits_end = first_ge(P.bwd_splits, 3, (int32_t)P.row_end);
  }
  v->num_local_items = (int64_t)P.dl_items.size() / 4;
  v->num_remote_items = (int64_t)P.dr_items.size() / 4;
  v->num_splits = (int64_t)P.d_splits.size() / 3;
  v->num_slots = P.n_d_slots;
  v->local_items = P.dl_items.data();
  v->remote_items = P.dr_items.data();
  v->splits = P.d_splits.data();
  return MEGA_OK;
}

mega_status mega_layout_device_bytes(const mega_layout *L, int32_t part, size_t *bytes) {
  clear_error();
  if (!L || !bytes) return fail(MEGA_ERR_INVALID_ARGUMENT, "null argument");
  if (part < 0 || part >= (int32_t)L->parts.size()) return fail(MEGA_ERR_INVALID_ARGUMENT, "part out of range");
  size_t offs[kImageArrays];
  *bytes = part_image_bytes(L, part, offs);
  return MEGA_OK;
}

mega_status mega_layout_bind_device(mega_layout *L, int32_t part, void *dev_buf, size_t bytes,
                                    mega_stream_t stream) {
  clear_error();
  if (!L || !dev_buf) return fail(MEGA_ERR_INVALID_ARGUMENT, "null argument");
  if (part < 0 || part >= (int32_t)L->parts.size()) return fail(MEGA_ERR_INVALID_ARGUMENT, "part out of range");
  if (reinterpret_cast<uintptr_t>(dev_buf) % 256) return fail(MEGA_ERR_INVALID_ARGUMENT, "dev_buf must be 256-byte aligned");
  size_t offs[kImageArrays];
  const size_t need = part_image_bytes(L, part, offs);
  if (bytes < need) return fail(MEGA_ERR_OUT_OF_MEMORY, "device buffer smaller than mega_layout_device_bytes");
  Part &P = L->parts[part];
  int dev = 0;
  cudaError_t ce = cudaGetDevice(&dev);
  if (ce != cudaSuccess) return fail(MEGA_ERR_CUDA, std::string("cudaGetDevice: ") + cudaGetErrorString(ce));
  // balanced chunks of work items (the kernels' schedule, see make_chunks)
  const std::vector<int32_t> fchunks = make_chunks(P.fwd_items, chunk_quantum(true), kChunkCapFwd);
  const std::vector<int32_t> bchunks = make_chunks(P.bwd_items, chunk_quantum(false), kChunkCapBwd);
  const std::vector<int32_t> none;
  if (L->parts.size() > 1) {
    dist_items(L, part, P.dl_items, P.dr_items, P.d_splits, P.n_d_slots);
    halo_plan(L, part, P.hsend_idx, P.hsend_off, P.hrecv_idx, P.hrecv_off, P.hpos);
  }
  // destination-pass row order.  The pass gathers nothing but streams each row's dz slice (16 B
  // per edge and head group) and its row operands.  When rows are long (mean in-degree >= 64) the
  // heavy rows (> 2x the mean) unbalance the static grid stride (a reddit hub carries ~40% of a
  // warp's share): they go first, longest first, the rest in layout order (reddit 1.40 -> 0.91
  // ms/step).  With short rows (products, mean 25) any reordering cost more than it balanced
  // (6.8 -> 7.8 ms/step measured), so the layout order is kept (no order array).
  std::vector<int32_t> dorder;
  {
    int64_t rows = (int64_t)P.indptr.size() - 1;
    const double mean = rows > 0 ? (double)P.indptr[rows] / (double)rows : 0.0;
    std::vector<int32_t> heavy;
    if (mean < 64.0) rows = 0;   // short rows: keep the layout order
    dorder.reserve(rows);
    for (int64_t r = 0; r < rows; ++r)
      if (P.indptr[r + 1] - P.indptr[r] > 2.0 * mean) heavy.push_back((int32_t)r);
    std::stable_sort(heavy.begin(), heavy.end(), [&](int32_t x, int32_t y) {
      return P.indptr[x + 1] - P.indptr[x] > P.indptr[y + 1] - P.indptr[y];
    });
    dorder = heavy;
    for (int64_t r = 0; r < rows; ++r)
      if (!(P.indptr[r + 1] - P.indptr[r] > 2.0 * mean)) dorder.push_back((int32_t)r);
  }
  const std::vector<int32_t> *arrs[kImageArrays] = {
      &P.indptr, &P.src, &P.cindptr, &P.cdst, &P.csr2csc, &P.fwd_items,
      &P.fwd_splits, &P.bwd_items, &P.bwd_splits, &fchunks, &bchunks, &none, &none, &P.cpos,
      &P.dl_items, &P.dr_items, &P.d_splits, &P.hsend_idx, &P.hrecv_idx, &P.hpos, &dorder};
  char *base = static_cast<char *>(dev_buf);
  for (int i = 0; i < kImageArrays; ++i) {
    if (arrs[i]->empty()) continue;
    ce = cudaMemcpyAsync(base + offs[i], arrs[i]->data(), arrs[i]->size() * sizeof(int32_t), cudaMemcpyHostToDevice,
                         (cudaStream_t)stream);
    if (ce != cudaSuccess) return fail(MEGA_ERR_CUDA, std::string("layout H2D copy: ") + cudaGetErrorString(ce));
  }
  P.device = dev;
  P.dev_base = dev_buf;
  DevPart &D = P.dev;
  D.indptr = reinterpret_cast<const int32_t *>(base + offs[0]);
  D.src = reinterpret_cast<const int32_t *>(base + offs[1]);
  D.cindptr = reinterpret_cast<const int32_t *>(base + offs[2]);
  D.cdst = reinterpret_cast<const int32_t *>(base + offs[3]);
  D.csr2csc = reinterpret_cast<const int32_t *>(base + offs[4]);
  D.fwd_items = reinterpret_cast<const int4 *>(base + offs[5]);
  D.fwd_splits = reinterpret_cast<const int32_t *>(base + offs[6]);
  D.bwd_items = reinterpret_cast<const int4 *>(base + offs[7]);
  D.bwd_splits = reinterpret_cast<const int32_t *>(base + offs[8]);
  D.fchunk = reinterpret_cast<const int32_t *>(base + offs[9]);
  D.bchunk = reinterpret_cast<const int32_t *>(base + offs[10]);
  D.cpos = reinterpret_cast<const int32_t *>(base + offs[13]);
  D.n_fchunks = (int32_t)fchunks.size() - 1;
  D.n_bchunks = (int32_t)bchunks.size() - 1;
  D.n = L->n;
  D.rows = P.row_end - P.row_begin;
  D.row_begin = P.row_begin;
  D.edges = (int64_t)P.src.size();
  D.n_fwd_items = (int32_t)(P.fwd_items.size() / 4);
  D.n_fwd_splits = (int32_t)(P.fwd_splits.size() / 3);
  D.n_fwd_slots = P.n_fwd_slots;
  D.n_bwd_items = (int32_t)(P.bwd_items.size() / 4);
  D.n_bwd_splits = (int32_t)(P.bwd_splits.size() / 3);
  D.n_bwd_slots = P.n_bwd_slots;
  D.id_mask = 0x7fffffffu;
  D.dl_items = reinterpret_cast<const int4 *>(base + offs[14]);
  D.dr_items = reinterpret_cast<const int4 *>(base + offs[15]);
  D.d_splits = reinterpret_cast<const int32_t *>(base + offs[16]);
  D.n_dl_items = (int32_t)(P.dl_items.size() / 4);
  D.n_dr_items = (int32_t)(P.dr_items.size() / 4);
  D.n_d_splits = (int32_t)(P.d_splits.size() / 3);
  D.n_d_slots = P.n_d_slots;
  D.hsend_idx = reinterpret_cast<const int32_t *>(base + offs[17]);
  D.hrecv_idx = reinterpret_cast<const int32_t *>(base + offs[18]);
  D.hpos = reinterpret_cast<const int32_t *>(base + offs[19]);
  D.dorder = dorder.empty() ? nullptr : reinterpret_cast<const int32_t *>(base + offs[20]);
  D.n_hsend = (int64_t)P.hsend_idx.size();
  D.n_hrecv = (int64_t)P.hrecv_idx.size();
  {  // own-source ranges of the CSC work (items and splits are sorted by source id)
    auto first_ge = [](const std::vector<int32_t> &v, int stride, int32_t x) {
      int64_t lo = 0, hi = (int64_t)v.size() / stride;
      while (lo < hi) { int64_t mid = (lo + hi) / 2; if (v[mid * stride] < x) lo = mid + 1; else hi = mid; }
      return (int32_t)lo;
    };
    D.bwd_own0 = first_ge(P.bwd_items, 4, (int32_t)P.row_begin);
    D.bwd_own1 = first_ge(P.bwd_items, 4, (int32_t)P.row_end);
    D.bsplit_own0 = first_ge(P.bwd_splits, 3, (int32_t)P.row_begin);
    D.bsplit_own1 = first_ge(P.bwd_splits, 3, (int32_t)P.row_end);
  }
  // pageable-memory copies return once staged, so the temporaries may go
  return MEGA_OK;
}

}  // extern "C"

// ---- persistence: "MEGALYT1" | version | sizes | arrays | fnv1a-64 checksum ----
namespace {
struct Writer {
  FILE *f;
  uint64_t h = 1469598103934665603ULL;
  bool ok = true;
  void raw(const void *p, size_t n) {
    const unsigned char *c = static_cast<const unsigned char *>(p);
    for (size_t i = 0; i < n; ++i) { h ^= c[i]; h *= 1099511628211ULL; }
    if (fwrite(p, 1, n, f) != n) ok = false;
  }
  template <typename T> void pod(const T &x) { raw(&x, sizeof x); }
  void vec(const std::vector<int32_t> &v) {
    uint64_t n = v.size();
    pod(n);
    if (n) raw(v.data(), n * sizeof(int32_t));
  }
};
struct Reader {
  FILE *f;
  uint64_t h = 1469598103934665603ULL;
  bool ok = true;
  void raw(void *p, size_t n) {
    if (fread(p, 1, n, f) != n) { ok = false; return; }
    const unsigned char *c = static_cast<const unsigned char *>(p);
    for (size_t i = 0; i < n; ++i) { h ^= c[i]; h *= 1099511628211ULL; }
  }
  template <typename T> void pod(T &x) { raw(&x, sizeof x); }
  void vec(std::vector<int32_t> &v) {
    uint64_t n = 0;
    pod(n);
    if (!ok || n > (1ULL << 34)) { ok = false; return; }
    v.resize(n);
    if (n) raw(v.data(), n * sizeof(int32_t));
  }
};
const char kMagic[8] = {'M', 'E', 'G', 'A', 'L', 'Y', 'T', '1'};
}  // namespace

extern "C" {

mega_status mega_layout_save(const mega_layout *L, const char *path) {
  clear_error();
  if (!L || !path) return fail(MEGA_ERR_INVALID_ARGUMENT, "null argument");
  FILE *f = fopen(path, "wb");
  if (!f) return fail(MEGA_ERR_IO, std::string("cannot open ") + path);
  Writer w{f};
  w.raw(kMagic, 8);
  int32_t ver = MEGA_ABI_VERSION;
  w.pod(ver);
  w.pod(L->n); w.pod(L->m); w.pod(L->opts); w.pod(L->stats);
  w.vec(L->perm); w.vec(L->new_of_old); w.vec(L->bounds);
  uint64_t k = L->parts.size();
  w.pod(k);
  for (const Part &P : L->parts) {
    w.pod(P.row_begin); w.pod(P.row_end); w.pod(P.n_fwd_slots); w.pod(P.n_bwd_slots);
    w.vec(P.indptr); w.vec(P.src); w.vec(P.eid); w.vec(P.cindptr); w.vec(P.cdst); w.vec(P.cpos);
    w.vec(P.csr2csc); w.vec(P.fwd_items); w.vec(P.fwd_splits); w.vec(P.bwd_items); w.vec(P.bwd_splits);
  }
  uint64_t sum = w.h;
  bool ok = w.ok && fwrite(&sum, sizeof sum, 1, f) == 1;
  ok = (fclose(f) == 0) && ok;
  return ok ? MEGA_OK : fail(MEGA_ERR_IO, "write failed");
}

mega_status mega_layout_load(const char *path, mega_layout **out) {
  clear_error();
  if (!path || !out) return fail(MEGA_ERR_INVALID_ARGUMENT, "null argument");
  *out = nullptr;
  FILE *f = fopen(path, "rb");
  if (!f) return fail(MEGA_ERR_IO, std::string("cannot open ") + path);
  mega_layout *L = new (std::nothrow) mega_layout();
  if (!L) { fclose(f); return fail(MEGA_ERR_OUT_OF_MEMORY, "layout allocation"); }
  Reader r{f};
  char magic[8];
  r.raw(magic, 8);
  int32_t ver = 0;
  r.pod(ver);
  if (!r.ok || std::memcmp(magic, kMagic, 8) != 0 || ver != MEGA_ABI_VERSION) {
    fclose(f); delete L;
    return fail(MEGA_ERR_IO, "not a MEGA layout file (magic/version)");
  }
  try {
    r.pod(L->n); r.pod(L->m); r.pod(L->opts); r.pod(L->stats);
    r.vec(L->perm); r.vec(L->new_of_old); r.vec(L->bounds);
    uint64_t k = 0;
    r.pod(k);
    if (!r.ok || k < 1 || k > 1024) throw 0;
    L->parts.resize(k);
    for (Part &P : L->parts) {
      r.pod(P.row_begin); r.pod(P.row_end); r.pod(P.n_fwd_slots); r.pod(P.n_bwd_slots);
      r.vec(P.indptr); r.vec(P.src); r.vec(P.eid); r.vec(P.cindptr); r.vec(P.cdst); r.vec(P.cpos);
      r.vec(P.csr2csc); r.vec(P.fwd_items); r.vec(P.fwd_splits); r.vec(P.bwd_items); r.vec(P.bwd_splits);
      if (!r.ok) throw 0;
      if (P.cindptr.size() != (size_t)L->n + 1 || P.indptr.empty()) throw 0;
      compute_class_histograms(P, L->n);
    }
  } catch (...) {
    fclose(f); delete L;
    return fail(MEGA_ERR_IO, "truncated or corrupt layout file");
  }
  uint64_t expect = r.h, sum = 0;
  bool ok = r.ok && fread(&sum, sizeof sum, 1, f) == 1 && sum == expect;
  fclose(f);
  if (!ok) { delete L; return fail(MEGA_ERR_IO, "layout file checksum mismatch"); }
  *out = L;
  return MEGA_OK;
}

}  // extern "C"
