// Device helpers and kernel argument blocks shared by the attention kernels
// (gat_kernels.cu).  Internal to libmega.so.
#pragma once
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <cmath>
#include <cstdint>

#include "mega_internal.h"

namespace mega {
namespace kern {

constexpr int MAXH = 8;
constexpr int WPB = 8;
constexpr int TPB = WPB * 32;
constexpr int MAX_GRID = 4096;


template <typename T> struct Tr;
template <> struct Tr<float> { static constexpr int EPV = 4; };
template <> struct Tr<__nv_bfloat16> { static constexpr int EPV = 8; };

// ---------------------------------------------------------------- loads
__device__ __forceinline__ uint64_t policy_last() {
  uint64_t p;
  asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ uint64_t policy_first() {
  uint64_t p;
  asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ uint64_t policy_normal() {
  uint64_t p;
  asm("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ uint4 ldg16(const void *p) { return __ldg(reinterpret_cast<const uint4 *>(p)); }
__device__ __forceinline__ uint4 ldg16_pol(const void *p, uint64_t pol) {
  uint4 r;
  asm("ld.global.nc.L2::cache_hint.v4.u32 {%0, %1, %2, %3}, [%4], %5;"
      : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
      : "l"(p), "l"(pol));
  return r;
}
// streamed index arrays: no L1 allocation, L2 evict_first
__device__ __forceinline__ int ld_stream(const int32_t *p, uint64_t pol) {
  int v;
  asm("ld.global.nc.L1::no_allocate.L2::cache_hint.b32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol));
  return v;
}
__device__ __forceinline__ void st16(void *p, uint4 v) { *reinterpret_cast<uint4 *>(p) = v; }
// streaming 16-byte stores with an L2 policy (evict_first: results written once must not push the
// gathered rows out of L2)
__device__ __forceinline__ void st16_pol(void *p, uint4 v, uint64_t pol) {
  asm volatile("st.global.L2::cache_hint.v4.u32 [%0], {%1, %2, %3, %4}, %5;" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z),
               "r"(v.w), "l"(pol)
               : "memory");
}
__device__ __forceinline__ void st16f_pol(void *p, float4 v, uint64_t pol) {
  st16_pol(p, make_uint4(__float_as_uint(v.x), __float_as_uint(v.y), __float_as_uint(v.z), __float_as_uint(v.w)), pol);
}

__device__ __forceinline__ void unpack(const uint4 &r, float (&x)[4], float) {
  x[0] = __uint_as_float(r.x); x[1] = __uint_as_float(r.y);
  x[2] = __uint_as_float(r.z); x[3] = __uint_as_float(r.w);
}
__device__ __forceinline__ void unpack(const uint4 &r, float (&x)[8], __nv_bfloat16) {
  x[0] = __uint_as_float(r.x << 16); x[1] = __uint_as_float(r.x & 0xffff0000u);
  x[2] = __uint_as_float(r.y << 16); x[3] = __uint_as_float(r.y & 0xffff0000u);
  x[4] = __uint_as_float(r.z << 16); x[5] = __uint_as_float(r.z & 0xffff0000u);
  x[6] = __uint_as_float(r.w << 16); x[7] = __uint_as_float(r.w & 0xffff0000u);
}
__device__ __forceinline__ uint32_t pk2(float a, float b) {
  __nv_bfloat162 t = __floats2bfloat162_rn(a, b);
  return *reinterpret_cast<uint32_t *>(&t);
}
__device__ __forceinline__ uint4 pack(const float (&x)[4], float) {
  return make_uint4(__float_as_uint(x[0]), __float_as_uint(x[1]), __float_as_uint(x[2]), __float_as_uint(x[3]));
}
__device__ __forceinline__ uint4 pack(const float (&x)[8], __nv_bfloat16) {
  return make_uint4(pk2(x[0], x[1]), pk2(x[2], x[3]), pk2(x[4], x[5]), pk2(x[6], x[7]));
}

template <int G> __device__ __forceinline__ float gmax(float v, unsigned mask) {
  if constexpr (G == 32) {   // whole warp: one CREDUX.MAX.F32 (sm_100a) instead of 5 shuffle + max steps
    float r;
    asm volatile("redux.sync.max.f32 %0, %1, 0xffffffff;" : "=f"(r) : "f"(v));
    return r;
  } else {
#pragma unroll
    for (int o = G / 2; o > 0; o >>= 1) v = fmaxf(v, __shfl_xor_sync(mask, v, o, G));
    return v;
  }
}
template <int G> __device__ __forceinline__ float gsum(float v, unsigned mask) {
#pragma unroll
  for (int o = G / 2; o > 0; o >>= 1) v += __shfl_xor_sync(mask, v, o, G);
  return v;
}
template <int HT> __device__ __forceinline__ float sel(const float (&a)[HT], int i) {
  float r = a[0];
#pragma unroll
  for (int h = 1; h < HT; ++h)
    if (i == h) r = a[h];
  return r;
}
// H (<= HT) consecutive fp32 values; 16-byte vectors when H % 4 == 0
template <int HT> __device__ __forceinline__ void load_h(const float *p, int H, float (&v)[HT]) {
  if (HT >= 4 && (H & 3) == 0) {
#pragma unroll
    for (int q = 0; q < HT / 4; ++q)
      if (4 * q < H) {
        float4 t = __ldg(reinterpret_cast<const float4 *>(p) + q);
        v[4 * q] = t.x; v[4 * q + 1] = t.y; v[4 * q + 2] = t.z; v[4 * q + 3] = t.w;
      }
  } else {
#pragma unroll
    for (int h = 0; h < HT; ++h)
      if (h < H) v[h] = __ldg(p + h);
  }
}
// volatile loads: issued exactly where written (software-pipelined prefetches)
__device__ __forceinline__ int ldv_i32(const int32_t *p, uint64_t pol) {
  int v;
  asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.b32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol));
  return v;
}
__device__ __forceinline__ int4 ldv_i4(const int4 *p) {
  int4 r;
  asm volatile("ld.global.nc.v4.s32 {%0, %1, %2, %3}, [%4];" : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}
__device__ __forceinline__ uint4 ldv16(const void *p) {
  uint4 r;
  asm volatile("ld.global.nc.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}
template <int HT> __device__ __forceinline__ void load_h_v(const float *p, int H, float (&v)[HT]) {
  if (HT >= 4 && (H & 3) == 0) {
#pragma unroll
    for (int q = 0; q < HT / 4; ++q)
      if (4 * q < H)
        asm volatile("ld.global.nc.v4.f32 {%0, %1, %2, %3}, [%4];"
                     : "=f"(v[4 * q]), "=f"(v[4 * q + 1]), "=f"(v[4 * q + 2]), "=f"(v[4 * q + 3])
                     : "l"(p + 4 * q));
  } else {
#pragma unroll
    for (int h = 0; h < HT; ++h)
      if (h < H) asm volatile("ld.global.nc.f32 %0, [%1];" : "=f"(v[h]) : "l"(p + h));
  }
}
// Packed fp32x2 FMA (sm_100 FFMA2): d{0,1} += a{0,1} * b, and the two-lane dot
// s{0,1} += a{0,1} * c{0,1}; halves the FMA issue count of the row loops.
__device__ __forceinline__ void ffma2s(float &d0, float &d1, float a0, float a1, float b) {
  unsigned long long D, A, B;
  asm("mov.b64 %0, {%1, %2};" : "=l"(A) : "f"(a0), "f"(a1));
  asm("mov.b64 %0, {%1, %2};" : "=l"(D) : "f"(d0), "f"(d1));
  asm("mov.b64 %0, {%1, %1};" : "=l"(B) : "f"(b));
  asm("fma.rn.f32x2 %0, %1, %2, %0;" : "+l"(D) : "l"(A), "l"(B));
  asm("mov.b64 {%0, %1}, %2;" : "=f"(d0), "=f"(d1) : "l"(D));
}
__device__ __forceinline__ void ffma2v(float &d0, float &d1, float a0, float a1, float c0, float c1) {
  unsigned long long D, A, C;
  asm("mov.b64 %0, {%1, %2};" : "=l"(A) : "f"(a0), "f"(a1));
  asm("mov.b64 %0, {%1, %2};" : "=l"(C) : "f"(c0), "f"(c1));
  asm("mov.b64 %0, {%1, %2};" : "=l"(D) : "f"(d0), "f"(d1));
  asm("fma.rn.f32x2 %0, %1, %2, %0;" : "+l"(D) : "l"(A), "l"(C));
  asm("mov.b64 {%0, %1}, %2;" : "=f"(d0), "=f"(d1) : "l"(D));
}
// exp / log on the SFU: ex2.approx / lg2.approx (max rel. error ~2^-22; the
// x*log2(e) rounding adds ~1e-7 |x| relative, within the fp32 parity bar)
__device__ __forceinline__ float fexp(float x) {
  float y;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x * 1.4426950408889634f));
  return y;
}
__device__ __forceinline__ float flog(float x) {
  float y;
  asm("lg2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y * 0.6931471805599453f;
}
__device__ __forceinline__ float leaky(float z, float slope) { return z > 0.f ? z : slope * z; }

// Sum per-vector partial dot products over the lanes (and vectors) of a head.
// LPH = lanes per head within one vector (head_dim / EPV), a compile-time
// power of two (heads is a power of two for every supported row width).
template <int G, int U, int V, int LPH>
__device__ __forceinline__ void head_reduce(float (&p)[U][V], unsigned mask) {
  if constexpr (LPH <= G) {
#pragma unroll
    for (int o = LPH >> 1; o > 0; o >>= 1) {
#pragma unroll
      for (int u = 0; u < U; ++u)
#pragma unroll
        for (int v = 0; v < V; ++v) p[u][v] += __shfl_xor_sync(mask, p[u][v], o, G);
    }
  } else {
    constexpr int VPH = LPH / G;
#pragma unroll
    for (int u = 0; u < U; ++u) {
      float q[V];
#pragma unroll
      for (int v = 0; v < V; ++v) {
        float t = 0.f;
#pragma unroll
        for (int v2 = 0; v2 < V; ++v2)
          if (v2 / VPH == v / VPH) t += p[u][v2];
        q[v] = t;
      }
#pragma unroll
      for (int v = 0; v < V; ++v) p[u][v] = gsum<G>(q[v], mask);
    }
  }
}
// Does this lane write the (reduced) value of vector v's head?
template <int G, int LPH>
__device__ __forceinline__ bool head_lead(int gl, int v) {
  if constexpr (LPH <= G) return (gl & (LPH - 1)) == 0;
  else return gl == 0 && (v % (LPH / G)) == 0;
}

// Reduce per-lane [V][EPV] accumulators over all groups of the block and store
// the block's [D] partial (fixed order -> deterministic; the cross-warp sum is
// carried in fp64 because these are long reductions with cancellation).
template <int G, int V, int EPV>
__device__ void block_partial(float (&acc)[V][EPV], double *s_red, double *dst, int D) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, gl = lane % G;
#pragma unroll
  for (int o = G; o < 32; o <<= 1)
#pragma unroll
    for (int v = 0; v < V; ++v)
#pragma unroll
      for (int k = 0; k < EPV; ++k) acc[v][k] += __shfl_xor_sync(0xffffffffu, acc[v][k], o);
  __syncthreads();
  for (int ww = 0; ww < WPB; ++ww) {
    if (w == ww && lane < G) {
#pragma unroll
      for (int v = 0; v < V; ++v)
#pragma unroll
        for (int k = 0; k < EPV; ++k) {
          const int col = (v * G + gl) * EPV + k;
          s_red[col] = (ww == 0 ? 0.0 : s_red[col]) + (double)acc[v][k];
        }
    }
    __syncthreads();
  }
  for (int d = threadIdx.x; d < D; d += TPB) dst[d] = s_red[d];
  __syncthreads();
}

// cp.async (LDGSTS) 16-byte copies with an L2 policy; commit / wait groups
__device__ __forceinline__ void cp_async16(void *smem, const void *gmem, uint64_t pol) {
  const uint32_t s = (uint32_t)__cvta_generic_to_shared(smem);
  asm volatile("cp.async.cg.shared.global.L2::cache_hint [%0], [%1], 16, %2;" ::"r"(s), "l"(gmem), "l"(pol)
               : "memory");
}
__device__ __forceinline__ void cp_async16_plain(void *smem, const void *gmem) {
  const uint32_t s = (uint32_t)__cvta_generic_to_shared(smem);
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(s), "l"(gmem) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N> __device__ __forceinline__ void cp_async_wait() {
  asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory");
}
// small cp.async staging copies (4 / 8 / 16 bytes, default L2 policy)
template <int B> __device__ __forceinline__ void cp_async_small(void *smem, const void *gmem) {
  const uint32_t s = (uint32_t)__cvta_generic_to_shared(smem);
  if constexpr (B == 16)
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(s), "l"(gmem) : "memory");
  else
    asm volatile("cp.async.ca.shared.global [%0], [%1], %2;" ::"r"(s), "l"(gmem), "n"(B) : "memory");
}
// H consecutive fp32 values (H a power of two <= 8, 4H-byte aligned) -> shared memory
template <int HT> __device__ __forceinline__ void cp_async_h(float *smem, const float *gmem) {
  if constexpr (HT == 8) {
    cp_async_small<16>(smem, gmem);
    cp_async_small<16>(smem + 4, gmem + 4);
  } else {
    cp_async_small<4 * HT>(smem, gmem);
  }
}
// per-thread prefetch of the 128-byte line holding p into L2
__device__ __forceinline__ void prefetch_l2_line(const void *p) {
  asm volatile("prefetch.global.L2 [%0];" ::"l"(p));
}
// TMA-engine prefetch of a contiguous range into L2 (no registers, no completion tracking)
__device__ __forceinline__ void prefetch_l2_bulk(const void *g, uint32_t bytes, uint64_t pol) {
  asm volatile("cp.async.bulk.prefetch.L2.global.L2::cache_hint [%0], %1, %2;" ::"l"(g), "r"(bytes), "l"(pol)
               : "memory");
}

struct FwdArgs {
  DevPart L;
  const void *feat;
  int64_t ldf;
  const float *el, *er;
  float *lse;
  int H, F, D;
  float slope;
  void *out;
  int64_t ldo;
  float *ws_m, *ws_l, *ws_acc;
  int st_hint;  // 1: streamed results (out rows) stored with L2 evict_first (MEGA_ST_HINT)
  int *ctr;     // zeroed work-claim counter (workspace), nullptr = static striding (MEGA_SCHED_DYN=0)
};

struct BwdArgs {
  DevPart L;
  const void *feat;
  int64_t ldf;
  const float *al, *ar;
  int H, F, D;
  float slope;
  const void *out;
  int64_t ldo;
  const void *gout;
  int64_t ldg;
  const float *el, *er, *lse;
  float *dlt, *der;
  float *gfeat;
  int64_t ldgf;
  void *gfeat_lp;
  int64_t ldlp;
  float *dz, *ws_bacc, *ws_bder;
  double *ws_dal, *ws_dar;
  float *gal, *gar;
  int nb_dst;
  int lp_only;     // MEGA_BWD_LP_ONLY: the final rows go to gfeat_lp only
  int lp_partial;  // (bf16, lp_only) the source pass's partial rows live in gfeat_lp too (no fp32 gfeat)
  int st_hint;  // 1: streamed results (dWh, dz, der) and the source's own Wh row use L2 evict_first
  int *ctr;     // zeroed work-claim counter of the source pass (workspace), nullptr = static striding
};

}  // namespace kern

}  // namespace mega
