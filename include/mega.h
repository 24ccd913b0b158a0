/*
 * mega.h — C ABI of libmega.so, the B200-native hot path of MEGA
 * (Deng & Rao, "MEGA: More Efficient Graph Attention for GNNs", ICDCS'24).
 * ABI version 2.  C linkage; plain pointers and sizes; no C++ or torch types.
 *
 * Citations "PAPER.md:L" are lines of the paper text;
 * DESIGN.md "Rn" are the documented readings of ambiguous passages.
 *
 * What the library computes (BASELINE.json north_star; GAT [14] cited at
 * PAPER.md:49; layer skeleton PAPER.md:51-55):
 *   a1  mega_preprocess   one traversal of the graph (Algorithm 1,
 *                         PAPER.md:239-306, reading R) -> node order -> an
 *                         exact relabelled layout (CSR, CSC, work items,
 *                         partitions) that preserves the edge multiset.
 *   a2  mega_project_fwd  Wh = X W (tensor cores), el = Wh.a_l, er = Wh.a_r.
 *   a3-a5 mega_gat_fwd    e_ij = LeakyReLU(a_l.Wh_i + a_r.Wh_j) for every edge
 *                         j->i, per-destination softmax, out_i = sum alpha Wh_j.
 *   a6-a8 mega_gat_bwd    gradients w.r.t. Wh, a_l, a_r.
 *   a9  mega_project_bwd  dW = X^T dWh, dX = dWh W^T.
 *
 * Conventions
 *   - Node ids: "new" ids are positions in the traversal order (perm[new] =
 *     old).  Every feature/ctx array passed to the compute calls is indexed
 *     by NEW ids; use mega_layout_view().perm to permute.
 *   - i = destination (CSR row, the aggregating node), j = source.  attn_l
 *     multiplies the DESTINATION row and attn_r the SOURCE row, exactly as
 *     north_star writes e_ij (DGL's GATConv names them the other way round).
 *   - Features are row-major [rows][ld] with D = heads*head_dim used columns,
 *     heads concatenated (column h*head_dim + f).  attn_l/attn_r are fp32
 *     [heads*head_dim] in the same column order.
 *   - ctx is an fp32 block of five planes [MEGA_CTX_PLANES][ctx_n][heads]:
 *     el, er, lse, Dlt, der, indexed by GLOBAL new node id (ctx_n =
 *     num_nodes).  lse = -inf for rows with no in-edges (whose out row is 0)
 *     (R6).  Dlt_i = g_i.out_i and der_j = sum over out-edges of
 *     dz are backward intermediates (der is a per-part partial for k > 1).
 *   - Multi-part layouts (num_parts = k > 1, destination-partitioned across k
 *     GPUs): part p owns rows [bounds[p], bounds[p+1]).  For
 *     part p, `out`, `grad_out` are LOCAL row arrays [rows_p][ld]; `feat`,
 *     `grad_feat` and ctx are GLOBAL [num_nodes].
 *   - Memory: the library never allocates device memory.  The caller owns
 *     every device buffer (the layout image, features, ctx, workspaces,
 *     outputs).  Host arrays passed in are read only during the call.
 *   - Streams: every device call is asynchronous and stream-ordered on the
 *     caller's stream (NULL = legacy default stream); the library never
 *     synchronises with the host unless MEGA_DEBUG_SYNC=1 is set in the
 *     environment (then every call synchronises and checks for faults).
 *   - Errors: every function returns mega_status; mega_last_error() gives a
 *     thread-local message for the last failure.  Arguments are validated on
 *     the host before any launch; outputs are unspecified after an error.
 *     Asynchronous device faults surface at the caller's next synchronisation.
 *   - Determinism: no atomics on any value path; results are bitwise
 *     reproducible run to run on the same GPU and layout.
 */
#ifndef MEGA_H
#define MEGA_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define MEGA_ABI_VERSION 2 /* 2: projection backward takes a workspace (tcgen05 dW split) */

typedef struct CUstream_st *mega_stream_t; /* == cudaStream_t */

typedef enum {
  MEGA_OK = 0,
  MEGA_ERR_INVALID_ARGUMENT = 1, /* null pointer, bad size, misaligned pointer/ld, bad dtype */
  MEGA_ERR_INVALID_GRAPH = 2,    /* indptr not monotone, indptr[n] != m, index out of range */
  MEGA_ERR_UNSUPPORTED = 3,      /* shape outside the kernels' supported set; device not sm_100 */
  MEGA_ERR_OUT_OF_MEMORY = 4,    /* host allocation failed, or a caller buffer is too small */
  MEGA_ERR_CUDA = 5,             /* a CUDA runtime / cuBLAS call failed (message has details) */
  MEGA_ERR_STATE = 6,            /* layout part not bound, or bound to another device */
  MEGA_ERR_IO = 7,               /* mega_layout_save / _load file errors or bad format */
  MEGA_ERR_NCCL = 8              /* NCCL could not be loaded or an NCCL call failed (message has details) */
} mega_status;

typedef enum { MEGA_F32 = 0, MEGA_BF16 = 1 } mega_dtype;

typedef enum {
  MEGA_ORDER_TRAVERSAL = 0, /* MEGA: traversal R of Algorithm 1 (the method) */
  MEGA_ORDER_IDENTITY = 1,  /* ablation: input order */
  MEGA_ORDER_DEGREE = 2,    /* ablation: stable sort by (-in-degree, id) */
  MEGA_ORDER_RANDOM = 3     /* ablation: Fisher-Yates on splitmix64(seed) */
} mega_order;

/* Input graph: CSR by destination.  Row i lists the sources j of the edges
 * j -> i (the paper's (v_src, v_dst) pairs).  Duplicate edges
 * and self-loops are allowed and kept (multiset semantics, R4/R5).
 * Requires 0 <= num_edges < 2^31 and 0 < num_nodes < 2^31. */
typedef struct {
  int64_t num_nodes;
  int64_t num_edges;
  const int64_t *indptr;  /* host [num_nodes + 1], indptr[0] = 0, monotone, indptr[n] = m */
  const int32_t *indices; /* host [num_edges], 0 <= j < num_nodes */
} mega_csr;

/* Schedule options.  Initialise with
 * mega_schedule_opts_init(); struct_size guards ABI evolution. */
typedef struct {
  uint32_t struct_size;
  int32_t window;        /* omega; 0 = auto clamp(round(m/n), 1, 64) */
  int32_t candidate_cap; /* K tier-1 candidates examined per step; 0 = 32 */
  int32_t order;         /* mega_order; non-TRAVERSAL orders exist for A/B ablations */
  int32_t seg_edges;     /* S: rows/sources with more edges are split into segments; 0 = auto */
  int32_t num_parts;     /* k >= 1 destination partitions (one per GPU) */
  uint64_t seed;         /* MEGA_ORDER_RANDOM only */
  /* L2 blocking (ours, not the paper's; R24): 0 = off.  B > 0 groups
   * the nodes into blocks of at most B nodes by size-constrained label
   * propagation on G_u, then stably sorts the order above by block (blocks
   * ranked by their first position in it), so the source rows one block of
   * destinations gathers fit the 126 MB L2.  Choose B ~ 0.4 * L2 bytes / row
   * bytes.  Each block keeps the traversal's order inside it. */
  int32_t block_rows;
  int32_t block_sweeps;  /* maximum label-propagation sweeps; 0 = 10 */
} mega_schedule_opts;

typedef struct mega_layout mega_layout;

typedef struct {
  uint32_t struct_size;
  int64_t num_nodes, num_edges, num_parts;
  int64_t window, candidate_cap, seg_edges, order;
  int64_t path_length; /* |P|: appearances incl. revisits */
  int64_t revisits;    /* |P| - n */
  int64_t jumps;       /* tier-3 picks after the start (virtual edges) */
  int64_t tile_unique_sources; /* sum over 64-row tiles of distinct sources (reuse = m / this) */
  int64_t max_in_degree, max_out_degree;
  double preprocess_seconds;
  int64_t block_rows;   /* B (0 = no L2 blocking) */
  int64_t num_blocks;   /* blocks after label propagation (1 per node with B = 1) */
  int64_t block_sweeps; /* sweeps run (stops early once a sweep changes < n/1000 labels) */
} mega_layout_stats;

/* Read-only host view of one part (for parity tests and for moving data into
 * the new order).  Pointers stay valid until mega_layout_destroy. */
typedef struct {
  uint32_t struct_size;
  int64_t num_nodes, num_edges; /* whole graph */
  int64_t row_begin, row_end;   /* rows of this part (new ids) */
  int64_t part_edges;
  int64_t num_fwd_items, num_fwd_splits, num_bwd_items, num_bwd_splits;
  int64_t num_parts;
  const int32_t *perm;       /* [num_nodes]   old id of new id */
  const int32_t *new_of_old; /* [num_nodes] */
  const int32_t *bounds;     /* [num_parts+1] row bounds of all parts */
  const int32_t *indptr;     /* [rows+1]  part-local CSR positions, rows sorted by (src, eid) */
  const int32_t *src;        /* [part_edges] new source id */
  const int32_t *eid;        /* [part_edges] position of the edge in the input CSR */
  const int32_t *cindptr;    /* [num_nodes+1] CSC over this part's edges, by new source id */
  const int32_t *cdst;       /* [part_edges] local destination row */
  const int32_t *cpos;       /* [part_edges] CSR position of CSC entry */
  const int32_t *csr2csc;    /* [part_edges] inverse of cpos */
  const int32_t *fwd_items;  /* [num_fwd_items][4] (row, e_begin, e_end, slot|-1) over CSR */
  const int32_t *fwd_splits; /* [num_fwd_splits][3] (row, first_slot, nseg) */
  const int32_t *bwd_items;  /* [num_bwd_items][4] over CSC rows (sources) */
  const int32_t *bwd_splits; /* [num_bwd_splits][3] */
} mega_layout_view;

#define MEGA_CTX_PLANES 5 /* el, er, lse, Dlt, der */

/* Flags */
#define MEGA_FLAG_ELER_IN_CTX 1u /* mega_gat_fwd: el/er planes of ctx are already valid (from
                                    mega_project_fwd); otherwise they are computed from feat */
#define MEGA_BWD_PHASE_SRC 2u    /* mega_gat_bwd: Dlt + source-major pass -> partial grad_feat and the
                                    der plane of ctx for ALL sources (k > 1: sum both over ranks onto
                                    the owners' rows before PHASE_DST) */
#define MEGA_BWD_PHASE_DST 4u    /* mega_gat_bwd: destination pass over this part's rows -> adds
                                    del_i a_l to grad_feat, writes grad_feat_lp, grad_attn_l and
                                    grad_attn_r (partials of this part for k > 1).  Neither flag = both. */
#define MEGA_DIST_PHASE_SEND 16u  /* mega_gat_*_dist: only the first half (see below); neither = both */
#define MEGA_DIST_PHASE_RECV 32u
#define MEGA_BWD_LP_ONLY 8u      /* mega_gat_bwd with grad_feat_lp != NULL: the final rows are written
                                    only to grad_feat_lp (the GEMM operand of mega_project_bwd);
                                    grad_feat keeps the fp32 source-phase partial.  Saves a D*4-byte
                                    write per row on the training path */

int mega_abi_version(void);
const char *mega_status_string(mega_status s);
const char *mega_last_error(void); /* thread-local; "" if none */
void mega_schedule_opts_init(mega_schedule_opts *opts);

/* a1. Reorganise (host, once per graph).  Traverses the graph once with
 * reading R of Algorithm 1 to get the node order,
 * then rewrites the CSR into the layout.  The edge
 * multiset is preserved exactly.  *out receives a new layout owned by the
 * caller (free with mega_layout_destroy).  Errors: INVALID_ARGUMENT (null,
 * opts), INVALID_GRAPH (CSR checks), OUT_OF_MEMORY. */
mega_status mega_preprocess(const mega_csr *csr, const mega_schedule_opts *opts, mega_layout **out);
void mega_layout_destroy(mega_layout *layout);
mega_status mega_layout_stats_get(const mega_layout *layout, mega_layout_stats *out);
mega_status mega_layout_view_get(const mega_layout *layout, int32_t part, mega_layout_view *out);

/* Persist / restore a layout (host part only; bind again after load).
 * Versioned little-endian binary with a checksum.  Errors: IO. */
mega_status mega_layout_save(const mega_layout *layout, const char *path);
mega_status mega_layout_load(const char *path, mega_layout **out);

/* Device image of one part: size, then an async H2D copy into a caller-owned
 * device buffer (>= bytes, 256-byte aligned) on `stream`, on the current
 * device.  The buffer must outlive every compute call on this part.  A part
 * may be re-bound (to another buffer or device).  Errors: INVALID_ARGUMENT,
 * OUT_OF_MEMORY (buffer too small), CUDA. */
mega_status mega_layout_device_bytes(const mega_layout *layout, int32_t part, size_t *bytes);
mega_status mega_layout_bind_device(mega_layout *layout, int32_t part, void *dev_buf, size_t bytes,
                                    mega_stream_t stream);

/* Workspace sizes (bytes, device) for mega_gat_fwd and mega_gat_bwd on a
 * part at this head shape and dtype. */
mega_status mega_gat_workspace_bytes(const mega_layout *layout, int32_t part, int heads, int head_dim,
                                     mega_dtype dtype, size_t *fwd_ws, size_t *bwd_ws);

/* a2. Projection (neural operator; the "sgemm" the paper finds
 * efficient): feat = x * w, then el = feat.a_l and er = feat.a_r
 * of every projected row into ctx rows [ctx_row0, ctx_row0+rows).
 *   MEGA_BF16: tcgen05 tensor-core GEMM (bf16 operands, fp32 accumulation in
 *     TMEM, TMA-staged operands); el/er are computed in its epilogue from the
 *     stored (bf16-rounded) feat.  Requires heads*head_dim a multiple of 64,
 *     head_dim a multiple of 8 dividing min(heads*head_dim, 256), in_dim, ldx and
 *     ldf multiples of 8, 16-byte aligned x, w, feat.
 *   MEGA_F32: true fp32 (no TF32) on CUDA cores (cuBLAS pedantic; the tensor
 *     cores have no fp32 kind), then an el/er pass.
 *   x    device [rows][ldx] dtype (columns >= in_dim are ignored),
 *   w    device [in_dim][heads*head_dim] dtype (dense rows),
 *   feat device [rows][ldf] dtype, ctx device fp32 [MEGA_CTX_PLANES][ctx_n][heads].
 * Errors: INVALID_ARGUMENT, UNSUPPORTED, CUDA. */
mega_status mega_project_fwd(const void *x, int64_t ldx, int64_t rows, int in_dim, const void *w, int heads,
                             int head_dim, const float *attn_l, const float *attn_r, mega_dtype dtype, void *feat,
                             int64_t ldf, float *ctx, int64_t ctx_n, int64_t ctx_row0, mega_stream_t stream);

/* Device workspace (bytes) of mega_project_bwd for this shape: the bf16 dW GEMM
 * is split over the rows (the reduction dimension) and its fp32 partial tiles
 * are summed in a fixed order (deterministic).  256 for MEGA_F32. */
mega_status mega_project_workspace_bytes(int64_t rows, int in_dim, int heads, int head_dim, mega_dtype dtype,
                                         size_t *bwd_ws);

/* a3-a5. Fused forward over `part`: per-edge score, per-destination online
 * softmax and attention-weighted aggregation, one pass over the edges
 * (PAPER.md:7, 84 — the irregular graph op the paper targets).
 *   feat  device [num_nodes][ldf] dtype (all sources, new order)
 *   out   device [rows_p][ldo] dtype  (written; 0 for rows without in-edges)
 *   ctx   device fp32 [MEGA_CTX_PLANES][num_nodes][heads]: writes lse (and
 *         el/er unless MEGA_FLAG_ELER_IN_CTX)
 *   ws    device, >= fwd_ws bytes from mega_gat_workspace_bytes.
 * Supported shapes: heads <= 8; head_dim a multiple of 8 (bf16) / 4 (fp32);
 * D/8 (bf16) or D/4 (fp32) a power of two <= 32 or a multiple of 32 up to 256;
 * ld*sizeof(dtype) a multiple of 16 and 16-byte aligned pointers.
 * Errors: INVALID_ARGUMENT, UNSUPPORTED, STATE (part not bound here), CUDA. */
mega_status mega_gat_fwd(const mega_layout *layout, int32_t part, const void *feat, int64_t ldf,
                         const float *attn_l, const float *attn_r, int heads, int head_dim, mega_dtype dtype,
                         float negative_slope, uint32_t flags, void *out, int64_t ldo, float *ctx, void *ws,
                         size_t ws_bytes, mega_stream_t stream);

/* a6-a8. Backward of mega_gat_fwd:
 *   Dlt_i = g_i.out_i; source-major pass over the CSC recomputing alpha and
 *   accumulating dWh_j = sum alpha g_i + der_j a_r, storing dz per edge;
 *   destination pass del_i = sum dz, dWh_i += del_i a_l.
 *   grad_out     device [rows_p][ldg] dtype
 *   grad_feat    device fp32 [num_nodes][ldgf] (written)
 *   grad_feat_lp optional device dtype [num_nodes][ldlp] copy of the final
 *                grad_feat rows of this part (operand of mega_project_bwd), or NULL
 *   grad_attn_l/r device fp32 [heads*head_dim] (written)
 * flags: MEGA_BWD_PHASE_* (see above).  Errors as mega_gat_fwd. */
mega_status mega_gat_bwd(const mega_layout *layout, int32_t part, const void *feat, int64_t ldf,
                         const float *attn_l, const float *attn_r, int heads, int head_dim, mega_dtype dtype,
                         float negative_slope, uint32_t flags, const void *out, int64_t ldo, const void *grad_out,
                         int64_t ldg, float *ctx, float *grad_feat, int64_t ldgf, void *grad_feat_lp,
                         int64_t ldlp, float *grad_attn_l, float *grad_attn_r, void *ws, size_t ws_bytes,
                         mega_stream_t stream);

/* a9. Projection backward: grad_w = x^T grad_feat (fp32 [in_dim][D], written)
 * and, if grad_x != NULL, grad_x = grad_feat w^T (dtype [rows][ldgx]).
 * MEGA_BF16: tcgen05 GEMMs (grad_feat is the bf16 copy, grad_feat_lp of
 * mega_gat_bwd); the dW partials use `ws` (>= mega_project_workspace_bytes).
 * MEGA_F32: fp32 on CUDA cores as in mega_project_fwd (ws unused).
 * Errors as mega_project_fwd, plus OUT_OF_MEMORY (workspace too small). */
mega_status mega_project_bwd(const void *x, int64_t ldx, int64_t rows, int in_dim, const void *w, int heads,
                             int head_dim, mega_dtype dtype, const void *grad_feat, int64_t ldgf, void *grad_x,
                             int64_t ldgx, float *grad_w, void *ws, size_t ws_bytes, mega_stream_t stream);

/* ---------------- k GPUs: destination partitions ----------------
 * The exact counterpart of the paper's "partition of the path representation
 * ... only two communications for adjacent path partitions":
 * a layout with num_parts = k gives rank p the contiguous, edge-balanced rows
 * [bounds[p], bounds[p+1]) of the MEGA order (R23) and every
 * in-edge of those rows.  Per layer, rank p exchanges the projected source
 * rows [Wh | er] in the forward and the partial [dWh | der] of other ranks'
 * rows in the backward.  The library owns the communicator. */
typedef struct mega_comm mega_comm;

/* NCCL transport (one process per GPU).  Rank 0 calls mega_comm_unique_id and
 * broadcasts the 128 bytes over the caller's own process group; every rank
 * then calls mega_comm_init with its rank and CUDA device.  libnccl.so.2 is
 * loaded on first use (the copy the process already has, else the system's).
 * Errors: NCCL (library missing or a call failed), CUDA, INVALID_ARGUMENT. */
mega_status mega_comm_unique_id(uint8_t id[128]);
mega_status mega_comm_init(const uint8_t id[128], int nranks, int rank, int device, mega_comm **out);
/* LOCAL transport: all `nranks` ranks driven by ONE process (devices[r], or
 * the current device for every rank when devices == NULL).  Messages are
 * stream-ordered device-to-device copies from the peer's buffers (peer
 * memory when ranks sit on different GPUs).  The caller runs every dist call
 * with MEGA_DIST_PHASE_SEND on all ranks, then with MEGA_DIST_PHASE_RECV on all
 * ranks, and must not modify a sent buffer until the receiving phase is done.
 * out[0..nranks) receive the communicators. */
mega_status mega_comm_init_local(int nranks, const int *devices, mega_comm **out);
void mega_comm_destroy(mega_comm *comm);
/* transport: 0 = NCCL, 1 = LOCAL */
mega_status mega_comm_info(const mega_comm *comm, int *nranks, int *rank, int *device, int *transport);

/* Read-only host view of the k-GPU work split of one part (for tests): the
 * forward items of the local pass (sources this part owns) and the remote pass,
 * as [n][4] (row, e_begin, e_end, slot | -1) over the part's CSR positions, the
 * merge records [n][3] (row, first_slot, nseg), and the ranges of bwd_items /
 * bwd_splits that belong to the part's own sources.  Empty for k = 1. */
typedef struct {
  uint32_t struct_size;
  int64_t num_local_items, num_remote_items, num_splits, num_slots;
  int64_t bwd_own_items_begin, bwd_own_items_end, bwd_own_splits_begin, bwd_own_splits_end;
  const int32_t *local_items, *remote_items, *splits;
  /* NEXT-1 halo plan: rows sent to / received from each peer (new ids, grouped by peer,
   * offsets [num_parts+1]); the forward moves these rows of [Wh | er] and the backward the
   * same rows of partial [dWh | der] the other way.  full_recv_rows = num_nodes - rows of
   * the part, what an all-gather would receive. */
  int64_t num_send, num_recv, full_recv_rows;
  const int32_t *send_idx, *send_off, *recv_idx, *recv_off;
} mega_layout_dist_view;
mega_status mega_layout_dist_view_get(mega_layout *layout, int32_t part, mega_layout_dist_view *out);

/* Workspaces of the dist calls on part `part` (fwd: slots of the split rows;
 * bwd: mega_gat_bwd's plus a receive area of (k-1) * rows_p * (D + heads) fp32). */
mega_status mega_gat_dist_workspace_bytes(const mega_layout *layout, int32_t part, int heads, int head_dim,
                                          mega_dtype dtype, size_t *fwd_ws, size_t *bwd_ws);

/* Forward on rank `part` (= the comm rank) of a k-part layout, overlapped with
 * the exchange (SURVEY §8(e) forward steps 2-4):
 *   1. on comm_stream: send this rank's projected rows [Wh | er] (feat rows and
 *      the er plane of ctx, rows [bounds[p], bounds[p+1])) to every peer and
 *      receive the peers' rows into the same global arrays;
 *   2. meanwhile on `stream`: fused score/softmax/aggregation over block (p,p),
 *      the in-edges whose source this rank owns;
 *   3. after the receives: the remote blocks, then a fixed-order merge (KB7) of
 *      the rows whose edges were split between the passes.
 * feat (device [num_nodes][ldf], GLOBAL rows, written for the peers' rows) must
 * hold this rank's projected rows; ctx holds their el/er with
 * MEGA_FLAG_ELER_IN_CTX (from mega_project_fwd), else they are computed first.
 * Other arguments as mega_gat_fwd.  PHASE flags: SEND = steps 1-2, RECV = step 3. */
mega_status mega_gat_fwd_dist(const mega_layout *layout, int32_t part, mega_comm *comm, void *feat, int64_t ldf,
                              const float *attn_l, const float *attn_r, int heads, int head_dim, mega_dtype dtype,
                              float negative_slope, uint32_t flags, void *out, int64_t ldo, float *ctx, void *ws,
                              size_t ws_bytes, mega_stream_t stream, mega_stream_t comm_stream);

/* Backward of mega_gat_fwd_dist (SURVEY §8(e) backward):
 *   SEND: Dlt; the source-major pass for the sources OTHER ranks own, whose
 *     partial [dWh | der] rows then travel to their owners on comm_stream
 *     (a reduce-scatter-v done as grouped point-to-point messages) while the
 *     source pass for this rank's own sources runs on `stream`;
 *   RECV: the peers' partials of this rank's rows are added in fixed peer
 *     order, then the destination pass on this rank's rows.
 * grad_feat: device fp32 [num_nodes][D] (ldgf == D), GLOBAL rows: on return
 * rows [bounds[p], bounds[p+1]) are final (other rows hold this rank's partial).
 * grad_attn_l/r are THIS RANK'S PARTIAL sums: the caller all-reduces them with
 * the projection's grad_w (data-parallel parameter gradients).
 * Other arguments as mega_gat_bwd. */
mega_status mega_gat_bwd_dist(const mega_layout *layout, int32_t part, mega_comm *comm, const void *feat,
                              int64_t ldf, const float *attn_l, const float *attn_r, int heads, int head_dim,
                              mega_dtype dtype, float negative_slope, uint32_t flags, const void *out, int64_t ldo,
                              const void *grad_out, int64_t ldg, float *ctx, float *grad_feat, int64_t ldgf,
                              void *grad_feat_lp, int64_t ldlp, float *grad_attn_l, float *grad_attn_r, void *ws,
                              size_t ws_bytes, mega_stream_t stream, mega_stream_t comm_stream);

/* NEXT-3: Graph Transformer edge attention, the paper's
 * headline model (Table I; DESIGN.md R-gt), over the same layout:
 *   s_e = Q_i.K_j / sqrt(head_dim) per head, alpha = softmax over In(i),
 *   out_i = sum_e alpha_e V_j.
 *   dtype  MEGA_F32: q/k/v/out fp32 (first cut: one warp per row and head);
 *          MEGA_BF16: q/k/v/out bf16 with fp32 accumulation (row-vector kernels
 *          over the layout's work items, split rows merged in fixed order;
 *          heads 1/2/4/8, head_dim a multiple of 8 with head_dim/8 a power of two,
 *          heads*head_dim/8 in {8, 16, 32, 64, 128}).
 *   q, k, v   device [num_nodes][ld] (new order; heads concatenated)
 *   out       device [rows_p][ldo] (written; 0 for rows without in-edges)
 *   lse       device fp32 [rows_p][heads] (written; -inf without in-edges)
 *   ws        device workspace >= mega_gt_workspace_bytes (unused by MEGA_F32 fwd).
 * Errors: INVALID_ARGUMENT, UNSUPPORTED, STATE (part not bound here), CUDA. */
mega_status mega_gt_workspace_bytes(const mega_layout *layout, int32_t part, int heads, int head_dim,
                                    mega_dtype dtype, size_t *ws_bytes);
mega_status mega_gt_fwd(const mega_layout *layout, int32_t part, const void *q, const void *k, const void *v,
                        int64_t ld, int heads, int head_dim, mega_dtype dtype, void *out, int64_t ldo, float *lse,
                        void *ws, size_t ws_bytes, mega_stream_t stream);

/* Backward of mega_gt_fwd, no atomics: destination pass over the CSR
 * (dQ_i = sum ds_e K_j / sqrt(F), ds_e = alpha_e (g_i.V_j - g_i.out_i), with
 * out the stored forward output), then source pass over the CSC
 * (dK_j = sum ds_e Q_i / sqrt(F), dV_j = sum alpha_e g_i).
 *   grad_out  device [rows_p][ldg] (dtype)
 *   grad_q    device fp32 [rows_p][ldgr] (written, this part's rows)
 *   grad_k/v  device fp32 [num_nodes][ldgr] (written; this part's partial
 *             when k > 1 — the caller sums over parts)
 * Errors as mega_gt_fwd, plus OUT_OF_MEMORY (workspace too small). */
mega_status mega_gt_bwd(const mega_layout *layout, int32_t part, const void *q, const void *k, const void *v,
                        int64_t ld, int heads, int head_dim, mega_dtype dtype, const void *out, int64_t ldo,
                        const float *lse, const void *grad_out, int64_t ldg, float *grad_q, float *grad_k,
                        float *grad_v, int64_t ldgr, void *ws, size_t ws_bytes, mega_stream_t stream);

/* Measurement helper (SURVEY §8(d)-d2 calibration; not part of the GAT path):
 * gathers the rows idx[0..n) of a device table [rows][row_bytes] (row_bytes in
 * {512, 1024, 2048}) on `stream`, XOR-folding them into `sink` (device fp32,
 * >= 64 * SM-count entries) so the loads cannot be elided.  Time it with CUDA
 * events to get the achievable row-gather bandwidth for an index pattern.
 * Errors: INVALID_ARGUMENT, UNSUPPORTED, OUT_OF_MEMORY (sink), CUDA. */
/* ---------------- NEXT-2: the faithful path-band representation ----------------
 * The paper's own layout (Fig. 7): traversal F of
 * Algorithm 1 (DESIGN.md R-band) builds a path P of node
 * appearances with revisits that covers every edge of the symmetrised simple
 * graph exactly once by a pair of appearances at most `window` apart (theta =
 * 1); the directed input multiset is stored on those pairs (multiplicities,
 * self-loops at a node's first appearance), so GAT over the band equals GAT
 * over the input (north_star).  Node ids are the INPUT ids (no relabelling).
 * Host build and view; the caller binds a device image like a layout. */
typedef struct mega_band mega_band;
typedef struct {
  uint32_t struct_size;
  int64_t num_nodes, num_edges, length; /* length = |P| */
  int32_t window, cap;
  int64_t jumps, virtual_edges, edges_u; /* tier-3 jumps, non-adjacent steps, |E_u| */
  int64_t num_slots, num_merges;         /* partial states of nodes appearing more than once */
  double build_seconds;
  const int32_t *P;             /* [length] input node id of each appearance */
  const uint64_t *own;          /* [length] bit o-1: edge {P[t], P[t-o]} covered when P[t] was appended */
  const uint64_t *lmask, *rmask;/* [length] bit o-1: an input edge P[t-o] -> P[t] / P[t+o] -> P[t] */
  const int32_t *cptr;          /* [length+1] offsets into cnt */
  const uint16_t *cnt;          /* multiplicities: lmask bits ascending, rmask bits, then self-loops */
  const int32_t *slot;          /* [length] partial slot or -1 */
  const int32_t *merges;        /* [num_merges][3] (node, first slot, count) */
} mega_band_view;
/* window 0 = auto clamp(round(m/n), 1, 64) (<= 64); cap 0 = 32.
 * Errors: INVALID_ARGUMENT, INVALID_GRAPH, UNSUPPORTED (a multiplicity > 65535), OUT_OF_MEMORY. */
mega_status mega_band_build(const mega_csr *csr, int32_t window, int32_t cap, mega_band **out);
void mega_band_destroy(mega_band *band);
mega_status mega_band_view_get(const mega_band *band, mega_band_view *out);
mega_status mega_band_device_bytes(const mega_band *band, size_t *bytes);
mega_status mega_band_bind_device(mega_band *band, void *dev_buf, size_t bytes, mega_stream_t stream);
/* GAT forward over the band: appearance tiles stream their window of rows
 * feat[P[t]] (t in [t0 - window, t1 + window)) into shared memory once and
 * aggregate each appearance's band in-edges from there (no per-edge gather);
 * nodes appearing more than once merge their appearances' partial softmax
 * states in fixed order.  feat / out device [num_nodes][ld] dtype (input
 * ids), rows of 32 x 16-byte vectors x V (bf16 D = 256 / 512 / 1024, fp32 D =
 * 128 / 256 / 512); el / er / lse: ctx planes as mega_gat_fwd (el / er
 * computed from feat unless MEGA_FLAG_ELER_IN_CTX); ws >= ws_bytes from
 * mega_band_gat_workspace_bytes.  Errors as mega_gat_fwd. */
mega_status mega_band_gat_workspace_bytes(const mega_band *band, int heads, int head_dim, mega_dtype dtype,
                                          size_t *ws_bytes);
mega_status mega_band_gat_fwd(const mega_band *band, const void *feat, int64_t ldf, const float *attn_l,
                              const float *attn_r, int heads, int head_dim, mega_dtype dtype, float negative_slope,
                              uint32_t flags, void *out, int64_t ldo, float *ctx, void *ws, size_t ws_bytes,
                              mega_stream_t stream);

/* Backward of mega_band_gat_fwd (a6-a8 on the band): Dlt per node; a source pass over
 * appearance tiles (window rows of grad_out staged in shared memory) accumulates each
 * appearance's share of sum alpha g_i and der_j and records c dz at each band entry; the
 * per-appearance del sums; a node pass sums a node's appearances in order and writes
 * grad_feat = sum alpha g + der a_r + del a_l (fp32 [num_nodes][ldgf]), the der plane
 * of ctx and fixed-order da_l / da_r.  out / grad_out: dtype [num_nodes][ld] (input
 * ids); ctx: as written by mega_band_gat_fwd; ws >= mega_band_gat_workspace_bytes.
 * Errors as mega_gat_bwd. */
mega_status mega_band_gat_bwd(const mega_band *band, const void *feat, int64_t ldf, const float *attn_l,
                              const float *attn_r, int heads, int head_dim, mega_dtype dtype, float negative_slope,
                              const void *out, int64_t ldo, const void *grad_out, int64_t ldg, float *ctx,
                              float *grad_feat, int64_t ldgf, float *grad_attn_l, float *grad_attn_r, void *ws,
                              size_t ws_bytes, mega_stream_t stream);

mega_status mega_calib_gather(const void *table, int64_t rows, int row_bytes, const int32_t *idx, int64_t n,
                              float *sink, int64_t sink_len, mega_stream_t stream);

#ifdef __cplusplus
}
#endif
#endif /* MEGA_H */
