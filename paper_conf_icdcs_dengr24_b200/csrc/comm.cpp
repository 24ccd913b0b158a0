// Multi-GPU exchange of the destination-partitioned path (
// PAPER.md:414 "only two communications for adjacent path partitions").
//
// A mega_comm is owned by the library and has one of two transports:
//   NCCL   one process per GPU (the production path, bench.py under torchrun):
//          a library-owned ncclComm_t, bootstrapped from a 128-byte unique id
//          that the caller broadcasts over its own process group.  libnccl is
//          dlopen'ed on first use (the one the process already loaded, e.g.
//          torch's, else the system's), so libmega.so has no link-time
//          dependency on it and loads on machines without NCCL.
//   LOCAL  every rank in ONE process (one GPU or several): sends are posted
//          as (device pointer, bytes, ready event) in a mailbox shared by the
//          group and receives are stream-ordered cudaMemcpyAsync copies from
//          the peer's buffer (peer memory over NVLink when the ranks sit on
//          different GPUs).  The driver calls each dist entry point with
//          MEGA_DIST_PHASE_SEND on every rank, then MEGA_DIST_PHASE_RECV on
//          every rank.  This is the k-part loopback used by the single-GPU
//          parity tests (SURVEY §8(e) "MEGA_LOOPBACK"), with the same kernels,
//          plans and buffers as the NCCL path; only the byte mover differs.
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <nccl.h>

#include <cstring>
#include <memory>
#include <mutex>
#include <string>
#include <vector>

#include "mega_internal.h"

namespace mega {
namespace {

struct NcclApi {
  bool ok = false;
  std::string err;
  ncclResult_t (*getUniqueId)(ncclUniqueId *) = nullptr;
  ncclResult_t (*commInitRank)(ncclComm_t *, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*commDestroy)(ncclComm_t) = nullptr;
  ncclResult_t (*groupStart)() = nullptr;
  ncclResult_t (*groupEnd)() = nullptr;
  ncclResult_t (*send)(const void *, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*recv)(void *, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  const char *(*errorString)(ncclResult_t) = nullptr;
};

const NcclApi &nccl() {
  static NcclApi api;
  static std::once_flag once;
  std::call_once(once, [] {
    void *h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL | RTLD_NOLOAD);
    if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
    if (!h) {
      const char *e = dlerror();
      api.err = std::string("cannot load libnccl.so.2: ") + (e ? e : "?");
      return;
    }
    auto sym = [&](const char *n) { return dlsym(h, n); };
    api.getUniqueId = reinterpret_cast<decltype(api.getUniqueId)>(sym("ncclGetUniqueId"));
    api.commInitRank = reinterpret_cast<decltype(api.commInitRank)>(sym("ncclCommInitRank"));
    api.commDestroy = reinterpret_cast<decltype(api.commDestroy)>(sym("ncclCommDestroy"));
    api.groupStart = reinterpret_cast<decltype(api.groupStart)>(sym("ncclGroupStart"));
    api.groupEnd = reinterpret_cast<decltype(api.groupEnd)>(sym("ncclGroupEnd"));
    api.send = reinterpret_cast<decltype(api.send)>(sym("ncclSend"));
    api.recv = reinterpret_cast<decltype(api.recv)>(sym("ncclRecv"));
    api.errorString = reinterpret_cast<decltype(api.errorString)>(sym("ncclGetErrorString"));
    api.ok = api.getUniqueId && api.commInitRank && api.commDestroy && api.groupStart && api.groupEnd && api.send &&
             api.recv && api.errorString;
    if (!api.ok) api.err = "libnccl.so.2 lacks a required symbol";
  });
  return api;
}

mega_status nccl_ok(ncclResult_t r, const char *what) {
  if (r == ncclSuccess) return MEGA_OK;
  return fail(MEGA_ERR_NCCL, std::string(what) + ": " + nccl().errorString(r));
}

}  // namespace

// Shared state of a LOCAL group: mailbox[src][dst][tag] = posted send.
struct LocalGroup {
  int k = 0;
  std::mutex mu;
  struct Post { const void *ptr = nullptr; size_t bytes = 0; cudaEvent_t ready = nullptr; bool valid = false; };
  std::vector<Post> box;  // [k][k][kTags]
  static constexpr int kTags = 8;
  Post &at(int s, int d, int tag) { return box[((size_t)s * k + d) * kTags + tag]; }
};

}  // namespace mega

struct mega_comm {
  int kind = 0;  // 0 = NCCL, 1 = LOCAL
  int nranks = 1, rank = 0, device = 0;
  ncclComm_t nc = nullptr;
  std::shared_ptr<mega::LocalGroup> grp;
  std::vector<cudaEvent_t> events;  // LOCAL: one per (peer, tag) send
  cudaEvent_t done = nullptr;       // end of the last exchange on the comm stream
};

namespace mega {

int comm_rank(const mega_comm *c) { return c->rank; }
int comm_size(const mega_comm *c) { return c->nranks; }
int comm_device(const mega_comm *c) { return c->device; }
bool comm_is_local(const mega_comm *c) { return c->kind == 1; }

// One exchange: `sends` and `recvs` are lists of (peer, tag, device pointer, bytes);
// NCCL matches the messages of a peer pair in order, LOCAL by tag.
// NCCL: one grouped send/recv on `cs` (both phases at once: NCCL needs every
// rank's sends and receives posted together).  LOCAL: PHASE_SEND posts the
// sends (after `ready_on` reaches this point), PHASE_RECV copies from the
// peers' posts on `cs`.  Afterwards `comm->done` marks completion on `cs`.
mega_status comm_exchange(mega_comm *c, const std::vector<CommMsg> &sends, const std::vector<CommMsg> &recvs,
                          cudaStream_t ready_on, cudaStream_t cs, bool phase_send, bool phase_recv) {
  cudaError_t ce;
  if (c->kind == 0) {
    if (!phase_send) return MEGA_OK;  // NCCL: everything was issued in the send phase
    // cs must see the data that ready_on produced
    if ((ce = cudaEventRecord(c->done, ready_on)) != cudaSuccess || (ce = cudaStreamWaitEvent(cs, c->done, 0)) != cudaSuccess)
      return fail(MEGA_ERR_CUDA, std::string("comm event: ") + cudaGetErrorString(ce));
    const NcclApi &N = nccl();
    mega_status rc = nccl_ok(N.groupStart(), "ncclGroupStart");
    if (rc != MEGA_OK) return rc;
    for (const CommMsg &m : sends)
      if (m.bytes && (rc = nccl_ok(N.send(m.ptr, m.bytes, ncclUint8, m.peer, c->nc, cs), "ncclSend")) != MEGA_OK) break;
    if (rc == MEGA_OK)
      for (const CommMsg &m : recvs)
        if (m.bytes && (rc = nccl_ok(N.recv(const_cast<void *>(m.ptr), m.bytes, ncclUint8, m.peer, c->nc, cs), "ncclRecv")) != MEGA_OK)
          break;
    mega_status rc2 = nccl_ok(N.groupEnd(), "ncclGroupEnd");
    if (rc != MEGA_OK) return rc;
    if (rc2 != MEGA_OK) return rc2;
    if ((ce = cudaEventRecord(c->done, cs)) != cudaSuccess) return fail(MEGA_ERR_CUDA, "comm done event");
    return MEGA_OK;
  }
  LocalGroup &G = *c->grp;
  for (const auto *L : {&sends, &recvs})
    for (const CommMsg &m : *L)
      if (m.tag < 0 || m.tag >= LocalGroup::kTags || m.peer < 0 || m.peer >= c->nranks || m.peer == c->rank)
        return fail(MEGA_ERR_INVALID_ARGUMENT, "comm message: bad peer or tag");
  if (phase_send) {
    std::lock_guard<std::mutex> g(G.mu);
    for (const CommMsg &m : sends) {
      LocalGroup::Post &p = G.at(c->rank, m.peer, m.tag);
      cudaEvent_t ev = c->events[(size_t)m.peer * LocalGroup::kTags + m.tag];
      if ((ce = cudaEventRecord(ev, ready_on)) != cudaSuccess)
        return fail(MEGA_ERR_CUDA, std::string("local post event: ") + cudaGetErrorString(ce));
      p.ptr = m.ptr; p.bytes = m.bytes; p.ready = ev; p.valid = true;
    }
  }
  if (phase_recv) {
    if ((ce = cudaEventRecord(c->done, ready_on)) != cudaSuccess || (ce = cudaStreamWaitEvent(cs, c->done, 0)) != cudaSuccess)
      return fail(MEGA_ERR_CUDA, std::string("comm event: ") + cudaGetErrorString(ce));
    std::lock_guard<std::mutex> g(G.mu);
    for (const CommMsg &m : recvs) {
      if (!m.bytes) continue;
      LocalGroup::Post &p = G.at(m.peer, c->rank, m.tag);
      if (!p.valid) return fail(MEGA_ERR_STATE, "LOCAL transport: peer " + std::to_string(m.peer) +
                                                    " has not posted its send (call PHASE_SEND on every rank first)");
      if (p.bytes != m.bytes) return fail(MEGA_ERR_STATE, "LOCAL transport: message size mismatch");
      if ((ce = cudaStreamWaitEvent(cs, p.ready, 0)) != cudaSuccess ||
          (ce = cudaMemcpyAsync(const_cast<void *>(m.ptr), p.ptr, m.bytes, cudaMemcpyDefault, cs)) != cudaSuccess)
        return fail(MEGA_ERR_CUDA, std::string("local copy: ") + cudaGetErrorString(ce));
      p.valid = false;
    }
    if ((ce = cudaEventRecord(c->done, cs)) != cudaSuccess) return fail(MEGA_ERR_CUDA, "comm done event");
  }
  return MEGA_OK;
}

cudaEvent_t comm_done_event(mega_comm *c) { return c->done; }

}  // namespace mega

using namespace mega;

extern "C" {

mega_status mega_comm_unique_id(uint8_t id[128]) {
  clear_error();
  if (!id) return fail(MEGA_ERR_INVALID_ARGUMENT, "null id");
  const NcclApi &N = nccl();
  if (!N.ok) return fail(MEGA_ERR_NCCL, N.err);
  static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId is 128 bytes");
  ncclUniqueId u;
  mega_status rc = nccl_ok(N.getUniqueId(&u), "ncclGetUniqueId");
  if (rc == MEGA_OK) std::memcpy(id, &u, 128);
  return rc;
}

static mega_status make_events(mega_comm *c) {
  cudaError_t ce = cudaEventCreateWithFlags(&c->done, cudaEventDisableTiming);
  if (ce != cudaSuccess) return fail(MEGA_ERR_CUDA, std::string("cudaEventCreate: ") + cudaGetErrorString(ce));
  if (c->kind == 1) {
    c->events.resize((size_t)c->nranks * LocalGroup::kTags);
    for (auto &e : c->events)
      if ((ce = cudaEventCreateWithFlags(&e, cudaEventDisableTiming)) != cudaSuccess)
        return fail(MEGA_ERR_CUDA, std::string("cudaEventCreate: ") + cudaGetErrorString(ce));
  }
  return MEGA_OK;
}

mega_status mega_comm_init(const uint8_t id[128], int nranks, int rank, int device, mega_comm **out) {
  clear_error();
  if (!id || !out || nranks < 1 || rank < 0 || rank >= nranks) return fail(MEGA_ERR_INVALID_ARGUMENT, "bad comm arguments");
  *out = nullptr;
  const NcclApi &N = nccl();
  if (!N.ok) return fail(MEGA_ERR_NCCL, N.err);
  cudaError_t ce = cudaSetDevice(device);
  if (ce != cudaSuccess) return fail(MEGA_ERR_CUDA, std::string("cudaSetDevice: ") + cudaGetErrorString(ce));
  auto c = std::make_unique<mega_comm>();
  c->kind = 0; c->nranks = nranks; c->rank = rank; c->device = device;
  ncclUniqueId u;
  std::memcpy(&u, id, 128);
  mega_status rc = nccl_ok(N.commInitRank(&c->nc, nranks, u, rank), "ncclCommInitRank");
  if (rc != MEGA_OK) return rc;
  if ((rc = make_events(c.get())) != MEGA_OK) return rc;
  *out = c.release();
  return MEGA_OK;
}

mega_status mega_comm_init_local(int nranks, const int *devices, mega_comm **out) {
  clear_error();
  if (!out || nranks < 1 || nranks > 1024) return fail(MEGA_ERR_INVALID_ARGUMENT, "bad comm arguments");
  auto grp = std::make_shared<LocalGroup>();
  grp->k = nranks;
  grp->box.resize((size_t)nranks * nranks * LocalGroup::kTags);
  int cur = 0;
  cudaGetDevice(&cur);
  for (int r = 0; r < nranks; ++r) out[r] = nullptr;
  for (int r = 0; r < nranks; ++r) {
    const int dev = devices ? devices[r] : cur;
    cudaError_t ce = cudaSetDevice(dev);
    if (ce != cudaSuccess) return fail(MEGA_ERR_CUDA, std::string("cudaSetDevice: ") + cudaGetErrorString(ce));
    auto c = std::make_unique<mega_comm>();
    c->kind = 1; c->nranks = nranks; c->rank = r; c->device = dev; c->grp = grp;
    mega_status rc = make_events(c.get());
    if (rc != MEGA_OK) { cudaSetDevice(cur); return rc; }
    out[r] = c.release();
  }
  cudaSetDevice(cur);
  return MEGA_OK;
}

void mega_comm_destroy(mega_comm *c) {
  if (!c) return;
  if (c->kind == 0 && c->nc && nccl().ok) nccl().commDestroy(c->nc);
  for (auto e : c->events) cudaEventDestroy(e);
  if (c->done) cudaEventDestroy(c->done);
  delete c;
}

mega_status mega_comm_info(const mega_comm *c, int *nranks, int *rank, int *device, int *transport) {
  clear_error();
  if (!c) return fail(MEGA_ERR_INVALID_ARGUMENT, "null comm");
  if (nranks) *nranks = c->nranks;
  if (rank) *rank = c->rank;
  if (device) *device = c->device;
  if (transport) *transport = c->kind;
  return MEGA_OK;
}

}  // extern "C"
