// Internal types of libmega.so (not part of the ABI).
#pragma once
#include <cstdint>
#include <string>
#include <vector>

#include <vector_types.h>

#include "../../include/mega.h"

namespace mega {

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
  int64_t n = 0, rows = 0, row_begin = 0, edges = 0;
  int32_t n_fwd_items = 0, n_fwd_splits = 0, n_fwd_slots = 0;
  int32_t n_bwd_items = 0, n_bwd_splits = 0, n_bwd_slots = 0;
};

struct Part {
  int64_t row_begin = 0, row_end = 0;
  std::vector<int32_t> indptr, src, eid, cindptr, cdst, cpos, csr2csc;
  std::vector<int32_t> fwd_items, fwd_splits, bwd_items, bwd_splits;
  int32_t n_fwd_slots = 0, n_bwd_slots = 0;
  // degrees sorted descending (host only): gather counts of source rows (out-degree in
  // this part) and destination rows (in-degree); used to pick L2-resident "hot" rows
  std::vector<int32_t> out_deg_desc, in_deg_desc;
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
size_t part_image_bytes(const mega_layout *L, int part, size_t offs[9]);
}  // namespace mega
