// a2 / a9: the dense node projection Wh = X W and its backward — the one real
// contraction of the path (north_star: tensor cores only here).
//   MEGA_BF16 (the training path bench.py times): hand-written tcgen05 GEMMs
//     (umma_gemm.cu: TMA -> shared memory -> tcgen05.mma -> TMEM), with el/er
//     computed in the forward GEMM's epilogue;
//   MEGA_F32 (the exact-arithmetic reference mode): the 5th-gen tensor cores
//     have no true-fp32 kind (kind::tf32 rounds operands to 10 bits), so this
//     mode keeps cuBLAS's CUBLAS_COMPUTE_32F_PEDANTIC GEMM (a plain library
//     GEMM on CUDA cores) followed by our el/er kernel (gat_kernels.cu).
#include <cublas_v2.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <mutex>
#include <unordered_map>

#include "mega_internal.h"

namespace mega {
mega_status launch_eler_any(mega_dtype dt, const void *feat, int64_t ldf, int64_t rows, int64_t row0, const float *al,
                            const float *ar, int heads, int head_dim, float *el, float *er, cudaStream_t st);
// umma_gemm.cu
mega_status umma_project_fwd(const void *x, int64_t ldx, int64_t rows, int in_dim, const void *w, int heads,
                             int head_dim, const float *al, const float *ar, void *feat, int64_t ldf, float *el,
                             float *er, int64_t ctx_row0, cudaStream_t st);
mega_status umma_project_dx(const void *gf, int64_t ldgf, int64_t rows, int in_dim, const void *w, int D, void *gx,
                            int64_t ldgx, cudaStream_t st);
void umma_dw_plan(int64_t rows, int in_dim, int D, int &splits, int64_t &mpad, size_t &bytes);
mega_status umma_project_dw(const void *x, int64_t ldx, const void *gf, int64_t ldgf, int64_t rows, int in_dim, int D,
                            float *gw, void *ws, size_t ws_bytes, cudaStream_t st);
namespace {

mega_status handle(cublasHandle_t &h) {
  static thread_local std::unordered_map<int, cublasHandle_t> hs;
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return fail(MEGA_ERR_CUDA, std::string("cudaGetDevice: ") + cudaGetErrorString(e));
  auto it = hs.find(dev);
  if (it == hs.end()) {
    cublasHandle_t nh;
    cublasStatus_t s = cublasCreate(&nh);
    if (s != CUBLAS_STATUS_SUCCESS) return fail(MEGA_ERR_CUDA, "cublasCreate failed (" + std::to_string((int)s) + ")");
    it = hs.emplace(dev, nh).first;
  }
  h = it->second;
  return MEGA_OK;
}

mega_status cublas_ok(cublasStatus_t s, const char *what) {
  if (s == CUBLAS_STATUS_SUCCESS) return MEGA_OK;
  return fail(MEGA_ERR_CUDA, std::string(what) + ": cuBLAS status " + std::to_string((int)s));
}

bool al16(const void *p) { return (reinterpret_cast<uintptr_t>(p) & 15) == 0; }

mega_status check_proj(const void *x, int64_t ldx, int64_t rows, int in_dim, const void *w, int heads, int head_dim,
                       mega_dtype dt) {
  if (!x || !w) return fail(MEGA_ERR_INVALID_ARGUMENT, "null pointer");
  if (dt != MEGA_F32 && dt != MEGA_BF16) return fail(MEGA_ERR_INVALID_ARGUMENT, "bad dtype");
  if (rows < 0 || in_dim < 1 || heads < 1 || head_dim < 1 || ldx < in_dim)
    return fail(MEGA_ERR_INVALID_ARGUMENT, "bad projection sizes");
  if (rows >= (1LL << 31)) return fail(MEGA_ERR_UNSUPPORTED, "rows must be < 2^31");
  int dev = 0, major = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, dev);
  if (major != 10) return fail(MEGA_ERR_UNSUPPORTED, "libmega.so requires an sm_100 (B200) device");
  if (dt == MEGA_BF16) {
    const int D = heads * head_dim;
    if (D % 64 || std::min(D, 256) % head_dim || head_dim % 8 || ldx % 8 ||
        (reinterpret_cast<uintptr_t>(x) & 15) || (reinterpret_cast<uintptr_t>(w) & 15))
      return fail(MEGA_ERR_UNSUPPORTED, "bf16 projection (tcgen05): heads*head_dim a multiple of 64, head_dim a "
                                        "multiple of 8 dividing min(D, 256), ldx a multiple of 8, "
                                        "16-byte aligned x and w");
  }
  return MEGA_OK;
}
}  // namespace
}  // namespace mega

using namespace mega;

extern "C" {

mega_status mega_project_fwd(const void *x, int64_t ldx, int64_t rows, int in_dim, const void *w, int heads,
                             int head_dim, const float *attn_l, const float *attn_r, mega_dtype dtype, void *feat,
                             int64_t ldf, float *ctx, int64_t ctx_n, int64_t ctx_row0, mega_stream_t stream) {
  clear_error();
  NvtxRange nvtx_("mega_project_fwd");
  mega_status rc = check_proj(x, ldx, rows, in_dim, w, heads, head_dim, dtype);
  if (rc != MEGA_OK) return rc;
  const int D = heads * head_dim;
  if (!feat || !ctx || !attn_l || !attn_r) return fail(MEGA_ERR_INVALID_ARGUMENT, "null pointer");
  if (ldf < D || ctx_row0 < 0 || ctx_row0 + rows > ctx_n) return fail(MEGA_ERR_INVALID_ARGUMENT, "bad ldf / ctx rows");
  if (!al16(feat) || !al16(ctx)) return fail(MEGA_ERR_INVALID_ARGUMENT, "feat/ctx must be 16-byte aligned");
  if (rows == 0) return MEGA_OK;
  cudaStream_t st = (cudaStream_t)stream;
  if (dtype == MEGA_BF16) {   // tcgen05 GEMM, el/er in its epilogue
    if (ldf % 8) return fail(MEGA_ERR_INVALID_ARGUMENT, "ldf must be a multiple of 8 (16-byte rows)");
    return umma_project_fwd(x, ldx, rows, in_dim, w, heads, head_dim, attn_l, attn_r, feat, ldf, ctx,
                            ctx + ctx_n * heads, ctx_row0, st);
  }
  cublasHandle_t h;
  if ((rc = handle(h)) != MEGA_OK) return rc;
  cublasSetStream(h, st);
  const float one = 1.f, zero = 0.f;
  // MEGA_F32: row-major Wh[rows][D] = X[rows][in] W[in][D]  <=>  col-major Wh^T = W^T X^T
  rc = cublas_ok(cublasGemmEx(h, CUBLAS_OP_N, CUBLAS_OP_N, D, (int)rows, in_dim, &one, w, CUDA_R_32F, D, x, CUDA_R_32F,
                              (int)ldx, &zero, feat, CUDA_R_32F, (int)ldf, CUBLAS_COMPUTE_32F_PEDANTIC,
                              CUBLAS_GEMM_DEFAULT),
                 "projection GEMM");
  if (rc != MEGA_OK) return rc;
  return launch_eler_any(dtype, feat, ldf, rows, ctx_row0, attn_l, attn_r, heads, head_dim, ctx,
                         ctx + ctx_n * heads, st);
}

mega_status mega_project_workspace_bytes(int64_t rows, int in_dim, int heads, int head_dim, mega_dtype dtype,
                                         size_t *bwd_ws) {
  clear_error();
  if (!bwd_ws || rows < 0 || in_dim < 1 || heads < 1 || head_dim < 1)
    return fail(MEGA_ERR_INVALID_ARGUMENT, "bad projection sizes");
  *bwd_ws = 256;
  if (dtype == MEGA_BF16 && rows > 0) {
    int splits;
    int64_t mpad;
    size_t b;
    umma_dw_plan(rows, in_dim, heads * head_dim, splits, mpad, b);
    *bwd_ws = b;
  }
  return MEGA_OK;
}

mega_status mega_project_bwd(const void *x, int64_t ldx, int64_t rows, int in_dim, const void *w, int heads,
                             int head_dim, mega_dtype dtype, const void *grad_feat, int64_t ldgf, void *grad_x,
                             int64_t ldgx, float *grad_w, void *ws, size_t ws_bytes, mega_stream_t stream) {
  clear_error();
  NvtxRange nvtx_("mega_project_bwd");
  mega_status rc = check_proj(x, ldx, rows, in_dim, w, heads, head_dim, dtype);
  if (rc != MEGA_OK) return rc;
  const int D = heads * head_dim;
  if (!grad_feat || !grad_w) return fail(MEGA_ERR_INVALID_ARGUMENT, "null pointer");
  if (ldgf < D || (grad_x && ldgx < in_dim)) return fail(MEGA_ERR_INVALID_ARGUMENT, "bad leading dimension");
  cudaStream_t st = (cudaStream_t)stream;
  if (rows == 0) return cudaMemsetAsync(grad_w, 0, sizeof(float) * (size_t)in_dim * D, st) == cudaSuccess
                            ? MEGA_OK : fail(MEGA_ERR_CUDA, "memset");
  if (dtype == MEGA_BF16) {   // tcgen05 GEMMs: dW split over rows (fixed-order reduce), dX
    if (ldgf % 8 || (grad_x && (ldgx % 8 || ldgx < (in_dim + 7) / 8 * 8)) || (reinterpret_cast<uintptr_t>(grad_feat) & 15) ||
        (grad_x && (reinterpret_cast<uintptr_t>(grad_x) & 15)))
      return fail(MEGA_ERR_INVALID_ARGUMENT, "bf16 projection backward: 16-byte rows and pointers");
    if (!ws) return fail(MEGA_ERR_INVALID_ARGUMENT, "null workspace (mega_project_workspace_bytes)");
    rc = umma_project_dw(x, ldx, grad_feat, ldgf, rows, in_dim, D, grad_w, ws, ws_bytes, st);
    if (rc != MEGA_OK || !grad_x) return rc;
    return umma_project_dx(grad_feat, ldgf, rows, in_dim, w, D, grad_x, ldgx, st);
  }
  cublasHandle_t h;
  if ((rc = handle(h)) != MEGA_OK) return rc;
  cublasSetStream(h, st);
  const float one = 1.f, zero = 0.f;
  const cublasComputeType_t ct = CUBLAS_COMPUTE_32F_PEDANTIC;
  // grad_w[in][D] = X^T dWh  <=>  col-major (D x in) = dWh^T(D x rows) * X(rows x in)
  rc = cublas_ok(cublasGemmEx(h, CUBLAS_OP_N, CUBLAS_OP_T, D, in_dim, (int)rows, &one, grad_feat, CUDA_R_32F, (int)ldgf,
                              x, CUDA_R_32F, (int)ldx, &zero, grad_w, CUDA_R_32F, D, ct, CUBLAS_GEMM_DEFAULT),
                 "grad_w GEMM");
  if (rc != MEGA_OK || !grad_x) return rc;
  // grad_x[rows][in] = dWh W^T  <=>  col-major (in x rows) = W(in x D, from row-major W^T) * dWh^T
  return cublas_ok(cublasGemmEx(h, CUBLAS_OP_T, CUBLAS_OP_N, in_dim, (int)rows, D, &one, w, CUDA_R_32F, D, grad_feat,
                                CUDA_R_32F, (int)ldgf, &zero, grad_x, CUDA_R_32F, (int)ldgx, ct, CUBLAS_GEMM_DEFAULT),
                   "grad_x GEMM");
}

}  // extern "C"
