// Internal types of libmega.so (not part of the ABI).
#pragma once
#include <cstdint>
#include <string>
#include <vector>

#include <cuda_runtime.h>
#include <nvtx3/nvToolsExt.h>
#include <vector_types.h>

#include "../../include/mega.h"

namespace mega {

// NVTX range around every C-ABI compute call (header-only NVTX3: a no-op unless a tool such as
// Nsight Systems / ncu --nvtx is attached), so profiles show the library calls by name.
struct NvtxRange {
  explicit NvtxRange(const char *name) { nvtxRangePushA(name); }
  ~NvtxRange() { nvtxRangePop(); }
  NvtxRange(const NvtxRange &) = delete;
  NvtxRange &operator=(const NvtxRange &) = delete;
};

// Sets the thread-local error message and returns the status.
mega_status fail(mega_status s, const std::string &msg);
void clear_error();

// Device pointers of one bound part (all int32; m < 2^31 is enforced).
struct DevPart {
  const int32_t *indptr = nullptr;   // [rows+1]
  const int32_t *src = nullptr;      // [E_p]
  const int32_t *cindptr = nullptr;  // [n+1]
  const int32_t *cdst = nullptr;     // [E_p]
  const int32_t *csr2csc = nullptr;  // [E_p]
  const int4 *fwd_items = nullptr;   // (row, e0, e1, slot)
  const int32_t *fwd_splits = nullptr;
  const int4 *bwd_items = nullptr;
  const int32_t *bwd_splits = nullptr;
  // balanced chunks of work items (make_chunks): chunk c = items [fchunk[c], fchunk[c+1]); a kernel's
  // group g takes chunks g, g + W, g + 2W, ... (W groups), so all groups advance through the layout
  // order at the same rate.  nullptr (the k-GPU passes over their own item lists): one item per chunk
  const int32_t *fchunk = nullptr;   // [n_fchunks + 1]
  const int32_t *bchunk = nullptr;   // [n_bchunks + 1]
  const int32_t *cpos = nullptr;      // [E_p] CSR position of each CSC edge (dz is stored in CSR order)
  const int32_t *dorder = nullptr;   // [rows] destination-pass row order: heavy rows first (see bind)
  int32_t n_fchunks = 0, n_bchunks = 0;
  int64_t n = 0, rows = 0, row_begin = 0, edges = 0;
  // id = entry & id_mask (round 1 packed a degree class into the high bits for L2 hints; now
  // plain ids, mask all ones)
  uint32_t id_mask = 0x7fffffffu;
  int32_t n_fwd_items = 0, n_fwd_splits = 0, n_fwd_slots = 0;
  int32_t n_bwd_items = 0, n_bwd_splits = 0, n_bwd_slots = 0;
  // k > 1 (destination-partitioned): the forward split by source owner.
  // Local pass items read only this part's own source rows (block (p,p)); remote pass
  // items the rest; rows with both (or long segments) go to slots merged by d_splits.
  const int4 *dl_items = nullptr, *dr_items = nullptr;
  const int32_t *d_splits = nullptr;
  int32_t n_dl_items = 0, n_dr_items = 0, n_d_splits = 0, n_d_slots = 0;
  // backward: items / splits of this part's own sources (rows [row_begin, row_end)) are the
  // contiguous ranges [bwd_own0, bwd_own1) of bwd_items and [bsplit_own0, bsplit_own1) of bwd_splits
  int32_t bwd_own0 = 0, bwd_own1 = 0, bsplit_own0 = 0, bsplit_own1 = 0;
  // NEXT-1 halo exchange: send_idx lists (peer by peer, ascending) the own rows some peer's edges
  // reference, recv_idx the peers' rows this part's edges reference; pos [k-1][rows] maps an own row
  // to the index of that peer's partial of it in the receive buffer (-1: the peer does not reference it)
  const int32_t *hsend_idx = nullptr, *hrecv_idx = nullptr, *hpos = nullptr;
  int64_t n_hsend = 0, n_hrecv = 0;
};

// NEXT-2 band layout, device pointers (band.cpp / band_kernels.cu)
struct BandDev {
  const int32_t *P = nullptr;                  // [L] node of each appearance
  const unsigned long long *lmask = nullptr;   // [L] bit o-1: in-edge from P[t-o]
  const unsigned long long *rmask = nullptr;   // [L] bit o-1: in-edge from P[t+o]
  const int32_t *cptr = nullptr;               // [L+1] offsets into cnt
  const uint16_t *cnt = nullptr;               // multiplicities (lmask bits, rmask bits, self-loops)
  const int32_t *slot = nullptr;               // [L] partial slot or -1
  const int32_t *merges = nullptr;             // [n_merges][3] (node, first slot, count)
  const int32_t *app_ptr = nullptr;            // [n+1] appearances of each node, in order
  const int32_t *app_idx = nullptr;            // [L]
  int64_t L = 0, n = 0, n_cnt = 0;
  int32_t omega = 0, n_merges = 0, n_slots = 0;
};

struct Part {
  int64_t row_begin = 0, row_end = 0;
  // k > 1 dist items (derived from indptr/src/bounds at bind time; host copies for the view)
  std::vector<int32_t> dl_items, dr_items, d_splits;
  int32_t n_d_slots = 0;
  std::vector<int32_t> hsend_idx, hsend_off, hrecv_idx, hrecv_off, hpos;   // halo plan (k > 1)
  std::vector<int32_t> indptr, src, eid, cindptr, cdst, cpos, csr2csc;
  std::vector<int32_t> fwd_items, fwd_splits, bwd_items, bwd_splits;
  int32_t n_fwd_slots = 0, n_bwd_slots = 0;
  // histograms of the degree classes (host only): how many source rows (by out-degree
  // in this part) / destination rows (by in-degree) fall in each class; used to pick
  // the L2-resident "hot" class threshold for a given row size
  int64_t out_cls[64] = {0}, in_cls[64] = {0};
  // binding
  int device = -1;
  void *dev_base = nullptr;
  DevPart dev;
};

}  // namespace mega

struct mega_layout {
  int64_t n = 0, m = 0;
  mega_schedule_opts opts{};
  mega_layout_stats stats{};
  std::vector<int32_t> perm, new_of_old, bounds;
  std::vector<mega::Part> parts;
};

namespace mega {
// preprocess.cpp
mega_status build_layout(const mega_csr *csr, const mega_schedule_opts *opts, mega_layout *L);
// image layout shared by device_bytes / bind
constexpr int kImageArrays = 21;
// dist items of part p (k > 1): see DevPart; S = the layout's segment size
void dist_items(const mega_layout *L, int part, std::vector<int32_t> &local, std::vector<int32_t> &remote,
                std::vector<int32_t> &splits, int32_t &nslots);
// NEXT-1 halo plan of part p (k > 1): rows each peer needs from p (send, grouped by peer q
// ascending, offsets [k+1]), rows p needs from each peer (recv), and p's pos map (see DevPart)
void halo_plan(const mega_layout *L, int part, std::vector<int32_t> &send_idx, std::vector<int32_t> &send_off,
               std::vector<int32_t> &recv_idx, std::vector<int32_t> &recv_off, std::vector<int32_t> &pos);
// comm.cpp: one exchange of (peer, pointer, bytes) messages (see mega_comm)
struct CommMsg { int peer; int tag; const void *ptr; size_t bytes; };
}  // namespace mega
struct mega_band;
namespace mega {
const BandDev *band_dev(const mega_band *B, int &device);
}  // namespace mega
struct mega_comm;
namespace mega {
int comm_rank(const mega_comm *c);
int comm_size(const mega_comm *c);
int comm_device(const mega_comm *c);
bool comm_is_local(const mega_comm *c);
mega_status comm_exchange(mega_comm *c, const std::vector<CommMsg> &sends, const std::vector<CommMsg> &recvs,
                          cudaStream_t ready_on, cudaStream_t cs, bool phase_send, bool phase_recv);
cudaEvent_t comm_done_event(mega_comm *c);
// Work schedule of the gathering kernels: consecutive work items (layout order) are grouped into
// chunks of about q edge-equivalents (each item costs its edges + kChunkItemCost), at most cap
// items (the forward stages one chunk's descriptors in one pass of its >= 8-lane groups).  With
// W groups taking chunks g, g + W, ..., every group gets the same work per round, so the groups
// stay within a few rounds of each other and the rows gathered concurrently stay in a narrow
// window of the order (L2 reuse).  q = 0: one item per chunk (plain item striding).
// MEGA_SCHED_Q / MEGA_SCHED_QB override q for the forward / source pass at bind time.
// Parts with fewer than kChunkMinItems work items keep one item per chunk: grouping a small graph's
// items would leave most of the grid idle (the paper's batches have ~1-5K items).
constexpr int kChunkItemCost = 2, kChunkEdgesFwd = 128, kChunkEdgesBwd = 128, kChunkCapFwd = 8, kChunkCapBwd = 1 << 30;
constexpr int64_t kChunkMinItems = 1 << 18;
std::vector<int32_t> make_chunks(const std::vector<int32_t> &items, int q, int cap);
size_t part_image_bytes(const mega_layout *L, int part, size_t offs[kImageArrays]);
// degree class: floor(2 log2 d) for d >= 1, clamped to 63; 0 for d = 0
inline int degree_class(int64_t d) {
  if (d <= 0) return 0;
  int k = 63 - __builtin_clzll((unsigned long long)d);
  int c = 2 * k + ((unsigned __int128)d * d >= ((unsigned __int128)1 << (2 * k + 1)) ? 1 : 0);
  return c > 63 ? 63 : c;
}
void compute_class_histograms(mega::Part &P, int64_t n);
}  // namespace mega
