// Graph Transformer edge attention over the MEGA layout (
// PAPER.md:94, Table I; DESIGN.md R-gt).  First correct cut, fp32:
//   s_e = Q_i.K_j / sqrt(F)   alpha = softmax over In(i)   out_i = sum alpha_e V_j
// The skeleton is the GAT path's (one warp per destination row and head, online
// softmax in registers; backward without atomics: destination pass over the CSR
// storing (alpha, ds) per edge, source pass over the CSC).  The per-edge score is
// an F-length dot product reduced across the warp.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <string>

#include "mega_internal.h"

namespace mega {
namespace gt {

constexpr int kMaxF = 128;            // head_dim <= 128: KF = ceil(F/32) <= 4 values per lane
constexpr int kWarps = 8;

struct Args {
  DevPart L;
  const float *q, *k, *v;
  int64_t ld;
  int H, F;
  float scale;                        // 1/sqrt(F)
  float *out; int64_t ldo;
  float *lse;                         // [rows][H]
  const float *outc; const float *lsec;
  const float *g; int64_t ldg;
  float *gq, *gk, *gv; int64_t ldgr;
  float *ws_alpha, *ws_ds;            // [E_p][H], CSR order
};

__device__ __forceinline__ float warp_sum(float x) {
#pragma unroll
  for (int o = 16; o; o >>= 1) x += __shfl_xor_sync(0xffffffffu, x, o);
  return x;
}

template <int KF>
__global__ void __launch_bounds__(kWarps * 32) gt_fwd_kernel(Args a) {
  const int lane = threadIdx.x & 31;
  const int64_t nw = (int64_t)gridDim.x * kWarps;
  const int64_t total = a.L.rows * a.H;
  for (int64_t w = (int64_t)blockIdx.x * kWarps + (threadIdx.x >> 5); w < total; w += nw) {
    const int64_t r = w / a.H;
    const int h = (int)(w - r * a.H);
    const int64_t i = a.L.row_begin + r;
    float q[KF], acc[KF];
#pragma unroll
    for (int t = 0; t < KF; ++t) {
      const int f = lane + 32 * t;
      q[t] = f < a.F ? a.q[i * a.ld + h * a.F + f] * a.scale : 0.f;
      acc[t] = 0.f;
    }
    float m = -INFINITY, S = 0.f;
    const int e0 = a.L.indptr[r], e1 = a.L.indptr[r + 1];
    int e = e0;
    for (; e + 1 < e1; e += 2) {    // two edges per iteration: both rows' loads in flight together
      const int64_t j0 = (int64_t)((uint32_t)a.L.src[e] & a.L.id_mask);
      const int64_t j1 = (int64_t)((uint32_t)a.L.src[e + 1] & a.L.id_mask);
      const float *k0 = a.k + j0 * a.ld + h * a.F, *k1 = a.k + j1 * a.ld + h * a.F;
      const float *v0 = a.v + j0 * a.ld + h * a.F, *v1 = a.v + j1 * a.ld + h * a.F;
      float p0 = 0.f, p1 = 0.f, w0[KF], w1[KF];
#pragma unroll
      for (int t = 0; t < KF; ++t) {
        const int f = lane + 32 * t;
        const bool ok = f < a.F;
        p0 += ok ? q[t] * k0[f] : 0.f;
        p1 += ok ? q[t] * k1[f] : 0.f;
        w0[t] = ok ? v0[f] : 0.f;
        w1[t] = ok ? v1[f] : 0.f;
      }
#pragma unroll
      for (int o = 16; o; o >>= 1) {
        p0 += __shfl_xor_sync(0xffffffffu, p0, o);
        p1 += __shfl_xor_sync(0xffffffffu, p1, o);
      }
      const float mn = fmaxf(m, fmaxf(p0, p1));
      const float c = __expf(m - mn), x0 = __expf(p0 - mn), x1 = __expf(p1 - mn);
      S = S * c + x0 + x1;
#pragma unroll
      for (int t = 0; t < KF; ++t) acc[t] = acc[t] * c + x0 * w0[t] + x1 * w1[t];
      m = mn;
    }
    for (; e < e1; ++e) {
      const int64_t j = (int64_t)((uint32_t)a.L.src[e] & a.L.id_mask);
      const float *kj = a.k + j * a.ld + h * a.F;
      const float *vj = a.v + j * a.ld + h * a.F;
      float part = 0.f, vv[KF];
#pragma unroll
      for (int t = 0; t < KF; ++t) {
        const int f = lane + 32 * t;
        part += f < a.F ? q[t] * kj[f] : 0.f;
        vv[t] = f < a.F ? vj[f] : 0.f;
      }
      const float s = warp_sum(part);
      const float mn = fmaxf(m, s);
      const float c = __expf(m - mn), p = __expf(s - mn);
      S = S * c + p;
#pragma unroll
      for (int t = 0; t < KF; ++t) acc[t] = acc[t] * c + p * vv[t];
      m = mn;
    }
    const float inv = S > 0.f ? 1.f / S : 0.f;
#pragma unroll
    for (int t = 0; t < KF; ++t) {
      const int f = lane + 32 * t;
      if (f < a.F) a.out[r * a.ldo + h * a.F + f] = acc[t] * inv;
    }
    if (lane == 0) a.lse[r * a.H + h] = S > 0.f ? m + __logf(S) : -INFINITY;
  }
}

// destination pass: Dlt_i = g_i.out_i; per in-edge alpha = exp(s - lse_i), dalpha = g_i.V_j,
// ds = alpha (dalpha - Dlt_i); dQ_i = sum ds K_j / sqrt(F); (alpha, ds) stored at the CSR position
template <int KF>
__global__ void __launch_bounds__(kWarps * 32) gt_bwd_dst_kernel(Args a) {
  const int lane = threadIdx.x & 31;
  const int64_t nw = (int64_t)gridDim.x * kWarps;
  const int64_t total = a.L.rows * a.H;
  for (int64_t w = (int64_t)blockIdx.x * kWarps + (threadIdx.x >> 5); w < total; w += nw) {
    const int64_t r = w / a.H;
    const int h = (int)(w - r * a.H);
    const int64_t i = a.L.row_begin + r;
    float q[KF], g[KF], dq[KF], dlt = 0.f;
#pragma unroll
    for (int t = 0; t < KF; ++t) {
      const int f = lane + 32 * t;
      const bool ok = f < a.F;
      q[t] = ok ? a.q[i * a.ld + h * a.F + f] * a.scale : 0.f;
      g[t] = ok ? a.g[r * a.ldg + h * a.F + f] : 0.f;
      dlt += ok ? g[t] * a.outc[r * a.ldo + h * a.F + f] : 0.f;
      dq[t] = 0.f;
    }
    dlt = warp_sum(dlt);
    const float lse = a.lsec[r * a.H + h];
    const int e0 = a.L.indptr[r], e1 = a.L.indptr[r + 1];
    for (int e = e0; e < e1; ++e) {
      const int64_t j = (int64_t)((uint32_t)a.L.src[e] & a.L.id_mask);
      const float *kj = a.k + j * a.ld + h * a.F;
      const float *vj = a.v + j * a.ld + h * a.F;
      float ps = 0.f, pd = 0.f, kk[KF];
#pragma unroll
      for (int t = 0; t < KF; ++t) {
        const int f = lane + 32 * t;
        kk[t] = f < a.F ? kj[f] : 0.f;
        ps += q[t] * kk[t];
        pd += f < a.F ? g[t] * vj[f] : 0.f;
      }
#pragma unroll
      for (int o = 16; o; o >>= 1) {
        ps += __shfl_xor_sync(0xffffffffu, ps, o);
        pd += __shfl_xor_sync(0xffffffffu, pd, o);
      }
      const float alpha = __expf(ps - lse);
      const float ds = alpha * (pd - dlt);
#pragma unroll
      for (int t = 0; t < KF; ++t) dq[t] += ds * kk[t];
      if (lane == 0) {
        a.ws_alpha[(int64_t)e * a.H + h] = alpha;
        a.ws_ds[(int64_t)e * a.H + h] = ds;
      }
    }
#pragma unroll
    for (int t = 0; t < KF; ++t) {
      const int f = lane + 32 * t;
      if (f < a.F) a.gq[r * a.ldgr + h * a.F + f] = dq[t] * a.scale;
    }
  }
}

// source pass over the CSC: dK_j = sum ds_e Q_i / sqrt(F), dV_j = sum alpha_e g_i (every source row written)
template <int KF>
__global__ void __launch_bounds__(kWarps * 32) gt_bwd_src_kernel(Args a) {
  const int lane = threadIdx.x & 31;
  const int64_t nw = (int64_t)gridDim.x * kWarps;
  const int64_t total = a.L.n * a.H;
  for (int64_t w = (int64_t)blockIdx.x * kWarps + (threadIdx.x >> 5); w < total; w += nw) {
    const int64_t j = w / a.H;
    const int h = (int)(w - j * a.H);
    float dk[KF], dv[KF];
#pragma unroll
    for (int t = 0; t < KF; ++t) dk[t] = dv[t] = 0.f;
    const int c0 = a.L.cindptr[j], c1 = a.L.cindptr[j + 1];
    for (int c = c0; c < c1; ++c) {
      const int64_t r = (int64_t)((uint32_t)a.L.cdst[c] & a.L.id_mask);
      const int64_t p = a.L.cpos[c];
      const float alpha = a.ws_alpha[p * a.H + h], ds = a.ws_ds[p * a.H + h];
      const float *qi = a.q + (a.L.row_begin + r) * a.ld + h * a.F;
      const float *gi = a.g + r * a.ldg + h * a.F;
#pragma unroll
      for (int t = 0; t < KF; ++t) {
        const int f = lane + 32 * t;
        if (f < a.F) {
          dk[t] += ds * qi[f];
          dv[t] += alpha * gi[f];
        }
      }
    }
#pragma unroll
    for (int t = 0; t < KF; ++t) {
      const int f = lane + 32 * t;
      if (f < a.F) {
        a.gk[j * a.ldgr + h * a.F + f] = dk[t] * a.scale;
        a.gv[j * a.ldgr + h * a.F + f] = dv[t];
      }
    }
  }
}

mega_status check(const mega_layout *L, int32_t part, int heads, int head_dim, int &sms, bool bf16 = false) {
  if (!L) return fail(MEGA_ERR_INVALID_ARGUMENT, "null layout");
  if (part < 0 || part >= (int32_t)L->parts.size()) return fail(MEGA_ERR_INVALID_ARGUMENT, "part out of range");
  if (heads < 1 || heads > 8 || head_dim < 1 || (!bf16 && head_dim > kMaxF))
    return fail(MEGA_ERR_UNSUPPORTED, "GT kernels: heads in [1, 8], head_dim in [1, 128] (fp32)");
  int dev = 0, major = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return fail(MEGA_ERR_CUDA, std::string("cudaGetDevice: ") + cudaGetErrorString(e));
  cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, dev);
  if (major != 10) return fail(MEGA_ERR_UNSUPPORTED, "libmega.so kernels require an sm_100 (B200) device");
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const Part &P = L->parts[part];
  if (!P.dev_base) return fail(MEGA_ERR_STATE, "layout part not bound (mega_layout_bind_device)");
  if (P.device != dev) return fail(MEGA_ERR_STATE, "layout part bound to another device");
  return MEGA_OK;
}

int grid_for(int64_t warps, int sms) {
  const int64_t blocks = (warps + kWarps - 1) / kWarps;
  const int64_t cap = (int64_t)sms * (2048 / (kWarps * 32));   // full occupancy, grid-stride beyond
  return (int)std::max<int64_t>(1, std::min(blocks, cap));
}

#define MEGA_GT_LAUNCH(KERNEL, warps)                                                   \
  do {                                                                                 \
    const int kf = (a.F + 31) / 32;                                                    \
    const int grid = gt::grid_for(warps, sms);                                             \
    if (grid > 0 && (warps) > 0) {                                                     \
      if (kf == 1) KERNEL<1><<<grid, gt::kWarps * 32, 0, st>>>(a);                         \
      else if (kf == 2) KERNEL<2><<<grid, gt::kWarps * 32, 0, st>>>(a);                    \
      else if (kf == 3) KERNEL<3><<<grid, gt::kWarps * 32, 0, st>>>(a);                    \
      else KERNEL<4><<<grid, gt::kWarps * 32, 0, st>>>(a);                                 \
      cudaError_t ce = cudaGetLastError();                                             \
      if (ce != cudaSuccess) return fail(MEGA_ERR_CUDA, std::string(#KERNEL ": ") + cudaGetErrorString(ce)); \
    }                                                                                  \
  } while (0)

}  // namespace gt
// gt_bf16.cu
size_t gtb_workspace_bytes(const Part &P, int H, int D);
mega_status gtb_run(const mega_layout *L, int32_t part, bool bwd, const void *q, const void *k, const void *v,
                    int64_t ld, int heads, int head_dim, void *out, int64_t ldo, float *lse, const void *grad_out,
                    int64_t ldg, float *gq, float *gk, float *gv, int64_t ldgr, void *ws, size_t ws_bytes,
                    cudaStream_t st, int sms);
}  // namespace mega

using namespace mega;

extern "C" {

mega_status mega_gt_workspace_bytes(const mega_layout *L, int32_t part, int heads, int head_dim, mega_dtype dtype,
                                    size_t *ws_bytes) {
  clear_error();
  if (!L || !ws_bytes) return fail(MEGA_ERR_INVALID_ARGUMENT, "null pointer");
  if (part < 0 || part >= (int32_t)L->parts.size()) return fail(MEGA_ERR_INVALID_ARGUMENT, "part out of range");
  if (heads < 1 || heads > 8 || head_dim < 1) return fail(MEGA_ERR_UNSUPPORTED, "heads in [1, 8]");
  if (dtype != MEGA_F32 && dtype != MEGA_BF16) return fail(MEGA_ERR_INVALID_ARGUMENT, "bad dtype");
  const Part &P = L->parts[part];
  if (dtype == MEGA_BF16) {
    *ws_bytes = gtb_workspace_bytes(P, heads, heads * head_dim);
    return MEGA_OK;
  }
  const size_t e = std::max<size_t>({(size_t)1, P.src.size(), (size_t)P.dev.edges});
  *ws_bytes = 2 * ((e * heads * 4 + 255) / 256 * 256);
  return MEGA_OK;
}

mega_status mega_gt_fwd(const mega_layout *L, int32_t part, const void *q_, const void *k_, const void *v_, int64_t ld,
                        int heads, int head_dim, mega_dtype dtype, void *out_, int64_t ldo, float *lse, void *ws,
                        size_t ws_bytes, mega_stream_t stream) {
  clear_error();
  NvtxRange nvtx_("mega_gt_fwd");
  int sms = 0;
  mega_status rc = gt::check(L, part, heads, head_dim, sms, dtype == MEGA_BF16);
  if (rc != MEGA_OK) return rc;
  if (!q_ || !k_ || !v_ || !out_ || !lse) return fail(MEGA_ERR_INVALID_ARGUMENT, "null pointer");
  const int64_t D = (int64_t)heads * head_dim;
  if (ld < D || ldo < D) return fail(MEGA_ERR_INVALID_ARGUMENT, "ld/ldo must be >= heads*head_dim");
  if (dtype == MEGA_BF16) {
    if (heads & (heads - 1)) return fail(MEGA_ERR_UNSUPPORTED, "bf16 GT: heads must be 1, 2, 4 or 8");
    if (!ws || ld % 8 || ldo % 8) return fail(MEGA_ERR_INVALID_ARGUMENT, "bf16 GT: workspace, 16-byte rows");
    return gtb_run(L, part, false, q_, k_, v_, ld, heads, head_dim, out_, ldo, lse, nullptr, 0, nullptr, nullptr,
                   nullptr, 0, ws, ws_bytes, (cudaStream_t)stream, sms);
  }
  if (dtype != MEGA_F32) return fail(MEGA_ERR_INVALID_ARGUMENT, "bad dtype");
  const float *q = static_cast<const float *>(q_), *k = static_cast<const float *>(k_),
              *v = static_cast<const float *>(v_);
  float *out = static_cast<float *>(out_);
  gt::Args a{};
  a.L = L->parts[part].dev;
  a.q = q; a.k = k; a.v = v; a.ld = ld;
  a.H = heads; a.F = head_dim; a.scale = 1.f / std::sqrt((float)head_dim);
  a.out = out; a.ldo = ldo; a.lse = lse;
  cudaStream_t st = (cudaStream_t)stream;
  MEGA_GT_LAUNCH(gt::gt_fwd_kernel, a.L.rows * heads);
  return MEGA_OK;
}

mega_status mega_gt_bwd(const mega_layout *L, int32_t part, const void *q_, const void *k_, const void *v_, int64_t ld,
                        int heads, int head_dim, mega_dtype dtype, const void *out_, int64_t ldo, const float *lse,
                        const void *grad_out_, int64_t ldg, float *grad_q, float *grad_k, float *grad_v, int64_t ldgr,
                        void *ws, size_t ws_bytes, mega_stream_t stream) {
  clear_error();
  NvtxRange nvtx_("mega_gt_bwd");
  int sms = 0;
  mega_status rc = gt::check(L, part, heads, head_dim, sms, dtype == MEGA_BF16);
  if (rc != MEGA_OK) return rc;
  if (!q_ || !k_ || !v_ || !out_ || !lse || !grad_out_ || !grad_q || !grad_k || !grad_v || !ws)
    return fail(MEGA_ERR_INVALID_ARGUMENT, "null pointer");
  const int64_t D = (int64_t)heads * head_dim;
  if (ld < D || ldo < D || ldg < D || ldgr < D) return fail(MEGA_ERR_INVALID_ARGUMENT, "leading dims must be >= D");
  if (dtype == MEGA_BF16) {
    if (heads & (heads - 1)) return fail(MEGA_ERR_UNSUPPORTED, "bf16 GT: heads must be 1, 2, 4 or 8");
    if (ld % 8 || ldo % 8 || ldg % 8 || ldgr % 4) return fail(MEGA_ERR_INVALID_ARGUMENT, "bf16 GT: 16-byte rows");
    return gtb_run(L, part, true, q_, k_, v_, ld, heads, head_dim, const_cast<void *>(out_), ldo,
                   const_cast<float *>(lse), grad_out_, ldg, grad_q, grad_k, grad_v, ldgr, ws, ws_bytes,
                   (cudaStream_t)stream, sms);
  }
  if (dtype != MEGA_F32) return fail(MEGA_ERR_INVALID_ARGUMENT, "bad dtype");
  const float *q = static_cast<const float *>(q_), *k = static_cast<const float *>(k_),
              *v = static_cast<const float *>(v_), *out = static_cast<const float *>(out_),
              *grad_out = static_cast<const float *>(grad_out_);
  size_t need = 0;
  mega_gt_workspace_bytes(L, part, heads, head_dim, MEGA_F32, &need);
  if (ws_bytes < need) return fail(MEGA_ERR_OUT_OF_MEMORY, "GT bwd workspace too small");
  gt::Args a{};
  a.L = L->parts[part].dev;
  a.q = q; a.k = k; a.v = v; a.ld = ld;
  a.H = heads; a.F = head_dim; a.scale = 1.f / std::sqrt((float)head_dim);
  a.outc = out; a.ldo = ldo; a.lsec = lse;
  a.g = grad_out; a.ldg = ldg;
  a.gq = grad_q; a.gk = grad_k; a.gv = grad_v; a.ldgr = ldgr;
  a.ws_alpha = static_cast<float *>(ws);
  a.ws_ds = reinterpret_cast<float *>(static_cast<char *>(ws) + need / 2);
  cudaStream_t st = (cudaStream_t)stream;
  MEGA_GT_LAUNCH(gt::gt_bwd_dst_kernel, a.L.rows * heads);
  MEGA_GT_LAUNCH(gt::gt_bwd_src_kernel, a.L.n * heads);
  return MEGA_OK;
}

}  // extern "C"
