// a2 / a9: the dense node projection Wh = X W and its backward — the one real
// contraction of the path (north_star: tensor cores only here).  This round
// the GEMMs go through cuBLAS (bf16 operands, fp32 accumulation, tensor
// cores; MEGA_F32 uses CUBLAS_COMPUTE_32F_PEDANTIC so no TF32), followed by
// our el/er kernel (gat_kernels.cu).  DESIGN.md "Projection" records the plan
// to replace this with a tcgen05 GEMM whose epilogue emits el/er.
#include <cublas_v2.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <mutex>
#include <unordered_map>

#include "mega_internal.h"

namespace mega {
mega_status launch_eler_any(mega_dtype dt, const void *feat, int64_t ldf, int64_t rows, int64_t row0, const float *al,
                            const float *ar, int heads, int head_dim, float *el, float *er, cudaStream_t st);
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
  mega_status rc = check_proj(x, ldx, rows, in_dim, w, heads, head_dim, dtype);
  if (rc != MEGA_OK) return rc;
  const int D = heads * head_dim;
  if (!feat || !ctx || !attn_l || !attn_r) return fail(MEGA_ERR_INVALID_ARGUMENT, "null pointer");
  if (ldf < D || ctx_row0 < 0 || ctx_row0 + rows > ctx_n) return fail(MEGA_ERR_INVALID_ARGUMENT, "bad ldf / ctx rows");
  if (!al16(feat) || !al16(ctx)) return fail(MEGA_ERR_INVALID_ARGUMENT, "feat/ctx must be 16-byte aligned");
  if (rows == 0) return MEGA_OK;
  cublasHandle_t h;
  if ((rc = handle(h)) != MEGA_OK) return rc;
  cudaStream_t st = (cudaStream_t)stream;
  cublasSetStream(h, st);
  const float one = 1.f, zero = 0.f;
  const cudaDataType_t T = dtype == MEGA_BF16 ? CUDA_R_16BF : CUDA_R_32F;
  const cublasComputeType_t ct = dtype == MEGA_BF16 ? CUBLAS_COMPUTE_32F : CUBLAS_COMPUTE_32F_PEDANTIC;
  // row-major Wh[rows][D] = X[rows][in] W[in][D]  <=>  col-major Wh^T = W^T X^T
  rc = cublas_ok(cublasGemmEx(h, CUBLAS_OP_N, CUBLAS_OP_N, D, (int)rows, in_dim, &one, w, T, D, x, T, (int)ldx, &zero,
                              feat, T, (int)ldf, ct, CUBLAS_GEMM_DEFAULT),
                 "projection GEMM");
  if (rc != MEGA_OK) return rc;
  return launch_eler_any(dtype, feat, ldf, rows, ctx_row0, attn_l, attn_r, heads, head_dim, ctx,
                         ctx + ctx_n * heads, st);
}

mega_status mega_project_bwd(const void *x, int64_t ldx, int64_t rows, int in_dim, const void *w, int heads,
                             int head_dim, mega_dtype dtype, const void *grad_feat, int64_t ldgf, void *grad_x,
                             int64_t ldgx, float *grad_w, mega_stream_t stream) {
  clear_error();
  mega_status rc = check_proj(x, ldx, rows, in_dim, w, heads, head_dim, dtype);
  if (rc != MEGA_OK) return rc;
  const int D = heads * head_dim;
  if (!grad_feat || !grad_w) return fail(MEGA_ERR_INVALID_ARGUMENT, "null pointer");
  if (ldgf < D || (grad_x && ldgx < in_dim)) return fail(MEGA_ERR_INVALID_ARGUMENT, "bad leading dimension");
  cublasHandle_t h;
  if ((rc = handle(h)) != MEGA_OK) return rc;
  cudaStream_t st = (cudaStream_t)stream;
  cublasSetStream(h, st);
  const float one = 1.f, zero = 0.f;
  const cudaDataType_t T = dtype == MEGA_BF16 ? CUDA_R_16BF : CUDA_R_32F;
  const cublasComputeType_t ct = dtype == MEGA_BF16 ? CUBLAS_COMPUTE_32F : CUBLAS_COMPUTE_32F_PEDANTIC;
  if (rows == 0) return cudaMemsetAsync(grad_w, 0, sizeof(float) * (size_t)in_dim * D, st) == cudaSuccess
                            ? MEGA_OK : fail(MEGA_ERR_CUDA, "memset");
  // grad_w[in][D] = X^T dWh  <=>  col-major (D x in) = dWh^T(D x rows) * X(rows x in)
  rc = cublas_ok(cublasGemmEx(h, CUBLAS_OP_N, CUBLAS_OP_T, D, in_dim, (int)rows, &one, grad_feat, T, (int)ldgf, x, T,
                              (int)ldx, &zero, grad_w, CUDA_R_32F, D, ct, CUBLAS_GEMM_DEFAULT),
                 "grad_w GEMM");
  if (rc != MEGA_OK || !grad_x) return rc;
  // grad_x[rows][in] = dWh W^T  <=>  col-major (in x rows) = W(in x D, from row-major W^T) * dWh^T
  return cublas_ok(cublasGemmEx(h, CUBLAS_OP_T, CUBLAS_OP_N, in_dim, (int)rows, D, &one, w, T, D, grad_feat, T,
                                (int)ldgf, &zero, grad_x, T, (int)ldgx, ct, CUBLAS_GEMM_DEFAULT),
                   "grad_x GEMM");
}

}  // extern "C"
