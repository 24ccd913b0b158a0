// NEXT-2: GAT forward over the faithful path-band layout (band.cpp; SURVEY §8(f),
// PAPER.md:188-235, 308-316).  The paper's point is that the band turns the
// neighbour gather into a sequential stream: appearance t's in-edges come from
// the appearances t - o and t + o, o <= omega.  Here a CTA takes a tile of T
// consecutive appearances, streams the rows feat[P[t']] of its window
// [t0 - omega, t0 + T + omega) into shared memory once (cp.async, 16-byte
// pieces), and each warp aggregates its appearances' band in-edges from there:
// the per-edge score (el of the destination, er of the window row), online
// softmax with multiplicities (p = count * exp(s - m)), weighted row sum —
// the arithmetic of gat_fwd_pipe_kernel (a 32-lane group per row, 16-byte
// vectors, packed FFMA2), with the row bytes read from shared memory instead
// of gathered.  A node appearing once writes its output row directly; the
// appearances of a node appearing more than once write partial softmax states
// that band_merge_kernel combines in appearance order (fixed order).
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>

#include "mega_internal.h"
#include "kern_common.cuh"

namespace mega {
mega_status launch_eler_any(mega_dtype dt, const void *feat, int64_t ldf, int64_t rows, int64_t row0, const float *al,
                            const float *ar, int heads, int head_dim, float *el, float *er, cudaStream_t st);
namespace kern {
namespace {

constexpr int BW = 8;              // warps per CTA
constexpr int BAND_SMEM = 100 * 1024;   // dynamic shared memory per CTA (two CTAs per SM)

struct BandArgs {
  BandDev B;
  const void *feat;
  int64_t ldf;
  const float *el, *er;
  float *lse;
  float slope;
  void *out;
  int64_t ldo;
  float *ws_m, *ws_l, *ws_acc;
  int D, T, win_cap;
  // backward
  const float *al, *ar;
  const void *gout;
  int64_t ldg;
  float *dlt, *der;                 // ctx planes (node ids)
  float *accD, *derp, *delp, *dzb;  // per appearance partials / per band entry c * dz
  float *gfeat;
  int64_t ldgf;
  double *pdal, *pdar;              // per-block partials of da_l / da_r
  float *gal, *gar;
};

__device__ __forceinline__ void *a256d(void *p) {   // 8-byte alignment for the mask arrays
  return reinterpret_cast<void *>((reinterpret_cast<uintptr_t>(p) + 7) & ~(uintptr_t)7);
}
// position (0-based) of the n-th set bit of a 64-bit mask
__device__ __forceinline__ int nth_bit64(unsigned long long m, int n) {
  const unsigned lo = (unsigned)m;
  const int c = __popc(lo);
  if (n < c) return (int)__fns(lo, 0, n + 1);
  return 32 + (int)__fns((unsigned)(m >> 32), 0, n - c + 1);
}

template <typename T, int V, int HT>
__global__ void __launch_bounds__(BW * 32, 2) band_fwd_kernel(const BandArgs a) {
  constexpr int G = 32, EPV = Tr<T>::EPV, FF = G * V * EPV / HT, SP = HT + 1, H = HT;
  extern __shared__ __align__(16) uint4 smem[];
  const int WC = a.win_cap;
  uint4 *rows = smem;                                                   // [WC][V * 32]
  float *er_w = reinterpret_cast<float *>(rows + (size_t)WC * V * 32);  // [WC][HT]
  int *p_w = reinterpret_cast<int *>(er_w + (size_t)WC * HT);           // [WC]
  __shared__ float s_p[BW][32][SP];
  __shared__ int s_w[BW][32];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  constexpr unsigned FULL = 0xffffffffu;
  const uint64_t pol_st = policy_first();
  int hv[V];
#pragma unroll
  for (int v = 0; v < V; ++v) hv[v] = ((v * G + lane) * EPV) / FF;
  const T *feat = static_cast<const T *>(a.feat);
  const int64_t L = a.B.L;
  const int om = a.B.omega;
  const int64_t ntiles = (L + a.T - 1) / a.T;
  for (int64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
    const int64_t t0 = tile * a.T, t1 = min(L, t0 + a.T);
    const int64_t wlo = max((int64_t)0, t0 - om), whi = min(L, t1 + om);
    const int nw = (int)(whi - wlo);
    __syncthreads();   // the previous tile's readers are done with the window
    for (int i = threadIdx.x; i < nw; i += blockDim.x) p_w[i] = a.B.P[wlo + i];
    __syncthreads();
    // the window: rows (each warp a row at a time, lane pieces) and er of every window row
    for (int i = w; i < nw; i += BW) {
      const T *rp = feat + (int64_t)p_w[i] * a.ldf + lane * EPV;
#pragma unroll
      for (int v = 0; v < V; ++v) cp_async16_plain(rows + ((size_t)i * V + v) * 32 + lane, rp + v * G * EPV);
    }
    cp_async_commit();
    for (int i = threadIdx.x; i < nw * H; i += blockDim.x) er_w[i] = a.er[(int64_t)p_w[i / H] * H + (i % H)];
    cp_async_wait<0>();
    __syncthreads();
    for (int64_t t = t0 + w; t < t1; t += BW) {
      const int ti = (int)(t - wlo);
      const int x = p_w[ti];
      const unsigned long long lm = a.B.lmask[t], rm = a.B.rmask[t];
      const int nl = __popcll(lm), nr = __popcll(rm);
      const int cb = a.B.cptr[t], ne = a.B.cptr[t + 1] - cb;   // nl + nr (+ 1 with self-loops)
      float elx[HT], mrun[HT], lrun[HT], acc[V][EPV];
      load_h<HT>(a.el + (int64_t)x * H, H, elx);
#pragma unroll
      for (int h = 0; h < HT; ++h) { mrun[h] = -INFINITY; lrun[h] = 0.f; }
#pragma unroll
      for (int v = 0; v < V; ++v)
#pragma unroll
        for (int k = 0; k < EPV; ++k) acc[v][k] = 0.f;
      for (int c0 = 0; c0 < ne; c0 += G) {
        const int e = c0 + lane;
        const bool valid = e < ne;
        int wi = ti;   // self-loop: the appearance's own row
        if (e < nl) wi = ti - (nth_bit64(lm, e) + 1);
        else if (e < nl + nr) wi = ti + (nth_bit64(rm, e - nl) + 1);
        const float mult = valid ? (float)a.B.cnt[cb + e] : 0.f;
        float sc[HT];
#pragma unroll
        for (int h = 0; h < HT; ++h) {
          const float s = valid ? leaky(elx[h] + er_w[wi * HT + h], a.slope) : -INFINITY;
          const float mn = fmaxf(mrun[h], gmax<G>(s, FULL));
          sc[h] = mn == -INFINITY ? 1.f : fexp(mrun[h] - mn);
          const float p = valid ? mult * fexp(s - mn) : 0.f;
          lrun[h] = fmaf(lrun[h], sc[h], p);
          mrun[h] = mn;
          s_p[w][lane][h] = p;
        }
        s_w[w][lane] = wi;
        if (c0 > 0) {
#pragma unroll
          for (int v = 0; v < V; ++v) {
            const float f = sel<HT>(sc, hv[v]);
#pragma unroll
            for (int k = 0; k < EPV; ++k) acc[v][k] *= f;
          }
        }
        __syncwarp();
        const int cnt = min(G, ne - c0);
        for (int k = 0; k < cnt; ++k) {
          const uint4 *rr = rows + (size_t)s_w[w][k] * V * 32 + lane;
#pragma unroll
          for (int v = 0; v < V; ++v) {
            const float pw = s_p[w][k][hv[v]];
            float xv[EPV];
            unpack(rr[v * 32], xv, T());
#pragma unroll
            for (int kk = 0; kk < EPV; kk += 2) ffma2s(acc[v][kk], acc[v][kk + 1], xv[kk], xv[kk + 1], pw);
          }
        }
        __syncwarp();
      }
      float lt[HT];
#pragma unroll
      for (int h = 0; h < HT; ++h) lt[h] = gsum<G>(lrun[h], FULL);
      const int slot = a.B.slot[t];
      if (slot < 0) {
        T *orow = static_cast<T *>(a.out) + (int64_t)x * a.ldo + lane * EPV;
#pragma unroll
        for (int v = 0; v < V; ++v) {
          const float Lh = sel<HT>(lt, hv[v]);
          const float inv = Lh > 0.f ? 1.f / Lh : 0.f;
          float y[EPV];
#pragma unroll
          for (int k = 0; k < EPV; ++k) y[k] = acc[v][k] * inv;
          st16_pol(orow + v * G * EPV, pack(y, T()), pol_st);
        }
        for (int h = lane; h < H; h += G) {
          const float Lh = sel<HT>(lt, h);
          a.lse[(int64_t)x * H + h] = Lh > 0.f ? sel<HT>(mrun, h) + flog(Lh) : -INFINITY;
        }
      } else {
        for (int h = lane; h < H; h += G) {
          a.ws_m[(int64_t)slot * H + h] = sel<HT>(mrun, h);
          a.ws_l[(int64_t)slot * H + h] = sel<HT>(lt, h);
        }
        float *pr = a.ws_acc + (int64_t)slot * a.D + lane * EPV;
#pragma unroll
        for (int v = 0; v < V; ++v)
#pragma unroll
          for (int k = 0; k < EPV; k += 4)
            *reinterpret_cast<float4 *>(pr + v * G * EPV + k) =
                make_float4(acc[v][k], acc[v][k + 1], acc[v][k + 2], acc[v][k + 3]);
      }
    }
  }
}

// The appearances of a node, merged in appearance order: M = max m_k, L = sum l_k e^{m_k - M},
// out = sum acc_k e^{m_k - M} / L, lse = M + log L (out = 0, lse = -inf without in-edges).
template <typename T, int V, int HT>
__global__ void __launch_bounds__(BW * 32) band_merge_kernel(const BandArgs a) {
  constexpr int G = 32, EPV = Tr<T>::EPV, FF = G * V * EPV / HT, H = HT;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  int hv[V];
#pragma unroll
  for (int v = 0; v < V; ++v) hv[v] = ((v * G + lane) * EPV) / FF;
  for (int64_t it = (int64_t)blockIdx.x * BW + w; it < a.B.n_merges; it += (int64_t)gridDim.x * BW) {
    const int x = a.B.merges[3 * it], s0 = a.B.merges[3 * it + 1], ns = a.B.merges[3 * it + 2];
    float M[HT], Ls[HT];
#pragma unroll
    for (int h = 0; h < HT; ++h) {
      M[h] = -INFINITY;
      for (int k = 0; k < ns; ++k) M[h] = fmaxf(M[h], a.ws_m[(int64_t)(s0 + k) * H + h]);
      Ls[h] = 0.f;
      if (M[h] != -INFINITY)
        for (int k = 0; k < ns; ++k) Ls[h] += a.ws_l[(int64_t)(s0 + k) * H + h] * fexp(a.ws_m[(int64_t)(s0 + k) * H + h] - M[h]);
    }
    for (int h = lane; h < H; h += G) {
      const float m_ = sel<HT>(M, h), l_ = sel<HT>(Ls, h);
      a.lse[(int64_t)x * H + h] = l_ > 0.f ? m_ + flog(l_) : -INFINITY;
    }
    T *orow = static_cast<T *>(a.out) + (int64_t)x * a.ldo;
#pragma unroll
    for (int v = 0; v < V; ++v) {
      const int col = (v * G + lane) * EPV;
      const float m_ = sel<HT>(M, hv[v]), l_ = sel<HT>(Ls, hv[v]);
      float y[EPV];
#pragma unroll
      for (int q = 0; q < EPV; ++q) y[q] = 0.f;
      if (l_ > 0.f) {
        for (int k = 0; k < ns; ++k) {
          const float f = fexp(a.ws_m[(int64_t)(s0 + k) * H + hv[v]] - m_);
          const float *pa = a.ws_acc + (int64_t)(s0 + k) * a.D + col;
#pragma unroll
          for (int q = 0; q < EPV; ++q) y[q] = fmaf(f, pa[q], y[q]);
        }
        const float inv = 1.f / l_;
#pragma unroll
        for (int q = 0; q < EPV; ++q) y[q] *= inv;
      }
      st16(orow + col, pack(y, T()));
    }
  }
}

// ---- backward over the band (SURVEY §8(a) a6-a8 on the band layout) ----
// Dlt_x = g_x . out_x per node (a6)
template <typename T, int V, int HT>
__global__ void __launch_bounds__(BW * 32) band_dlt_kernel(const BandArgs a) {
  constexpr int G = 32, EPV = Tr<T>::EPV, FF = G * V * EPV / HT, LPH = FF / EPV, H = HT;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  for (int64_t x = (int64_t)blockIdx.x * BW + w; x < a.B.n; x += (int64_t)gridDim.x * BW) {
    const T *gr = static_cast<const T *>(a.gout) + x * a.ldg + lane * EPV;
    const T *orr = static_cast<const T *>(a.out) + x * a.ldo + lane * EPV;
#pragma unroll
    for (int v = 0; v < V; ++v) {
      float xg[EPV], xo[EPV];
      unpack(ldg16(gr + v * G * EPV), xg, T());
      unpack(ldg16(orr + v * G * EPV), xo, T());
      float d = 0.f;
#pragma unroll
      for (int k = 0; k < EPV; ++k) d = fmaf(xg[k], xo[k], d);
      if constexpr (LPH >= G) {
        d = gsum<G>(d, 0xffffffffu);
      } else {
#pragma unroll
        for (int o = LPH / 2; o > 0; o >>= 1) d += __shfl_xor_sync(0xffffffffu, d, o);
      }
      // a head may span several vectors (LPH > G): sum over v of the head in registers
      const int h = ((v * G + lane) * EPV) / FF;
      if constexpr (LPH > G) {
        __shared__ float s_acc[BW][HT];
        if (lane == 0) s_acc[w][h] = (v % (LPH / G) == 0 ? 0.f : s_acc[w][h]) + d;
        __syncwarp();
        if (lane == 0 && (v % (LPH / G)) == LPH / G - 1) a.dlt[x * H + h] = s_acc[w][h];
        __syncwarp();
      } else {
        if ((lane % LPH) == 0) a.dlt[x * H + h] = d;
      }
    }
  }
}

// Source pass (a7) over appearance tiles: appearance t is source j = P[t] of the band edges
// t -> t + o (lmask[t+o] bit o-1), t -> t - o (rmask[t-o] bit o-1) and its own self-loops; the window
// rows g[P[t']] and (el, lse, Dlt)[P[t']] are staged in shared memory.  Per appearance:
// accD[t] = sum c alpha g_i, derp[t] = sum c dz; c dz is stored at the edge's band entry (dzb).
template <typename T, int V, int HT>
__global__ void __launch_bounds__(BW * 32, 2) band_src_kernel(const BandArgs a) {
  constexpr int G = 32, EPV = Tr<T>::EPV, FF = G * V * EPV / HT, LPH = FF / EPV, H = HT;
  extern __shared__ __align__(16) uint4 smem[];
  const int WC = a.win_cap;
  uint4 *rows = smem;                                                     // [WC][V * 32] g rows
  float *eld = reinterpret_cast<float *>(rows + (size_t)WC * V * 32);     // [WC][3][HT] el, lse, Dlt
  int *p_w = reinterpret_cast<int *>(eld + (size_t)WC * 3 * HT);          // [WC]
  unsigned long long *lm_w = reinterpret_cast<unsigned long long *>(a256d(p_w + WC));  // [WC]
  unsigned long long *rm_w = lm_w + WC;                                   // [WC]
  int *cp_w = reinterpret_cast<int *>(rm_w + WC);                         // [WC + 1]
  __shared__ int s_wi[BW][32], s_pos[BW][32];
  __shared__ float s_c[BW][32];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  constexpr unsigned FULL = 0xffffffffu;
  int hv[V];
#pragma unroll
  for (int v = 0; v < V; ++v) hv[v] = ((v * G + lane) * EPV) / FF;
  const T *feat = static_cast<const T *>(a.feat);
  const T *gout = static_cast<const T *>(a.gout);
  const int64_t L = a.B.L;
  const int om = a.B.omega;
  const int64_t ntiles = (L + a.T - 1) / a.T;
  for (int64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
    const int64_t t0 = tile * a.T, t1 = min(L, t0 + a.T);
    const int64_t wlo = max((int64_t)0, t0 - om), whi = min(L, t1 + om);
    const int nw = (int)(whi - wlo);
    __syncthreads();
    for (int i = threadIdx.x; i < nw; i += blockDim.x) {
      p_w[i] = a.B.P[wlo + i];
      lm_w[i] = a.B.lmask[wlo + i];
      rm_w[i] = a.B.rmask[wlo + i];
      cp_w[i] = a.B.cptr[wlo + i];
    }
    if (threadIdx.x == 0) cp_w[nw] = a.B.cptr[whi];
    __syncthreads();
    for (int i = w; i < nw; i += BW) {
      const T *rp = gout + (int64_t)p_w[i] * a.ldg + lane * EPV;
#pragma unroll
      for (int v = 0; v < V; ++v) cp_async16_plain(rows + ((size_t)i * V + v) * 32 + lane, rp + v * G * EPV);
    }
    cp_async_commit();
    for (int i = threadIdx.x; i < nw * 3 * H; i += blockDim.x) {
      const int r = i / (3 * H), q = (i / H) % 3, h = i % H;
      const float *src = q == 0 ? a.el : (q == 1 ? a.lse : a.dlt);
      eld[i] = src[(int64_t)p_w[r] * H + h];
    }
    cp_async_wait<0>();
    __syncthreads();
    for (int64_t t = t0 + w; t < t1; t += BW) {
      const int ti = (int)(t - wlo);
      const int j = p_w[ti];
      float whf[V][EPV], acc[V][EPV], erj[HT], dsum[HT];
      {
        const T *rp = feat + (int64_t)j * a.ldf + lane * EPV;
#pragma unroll
        for (int v = 0; v < V; ++v) {
          unpack(ldg16(rp + v * G * EPV), whf[v], T());
#pragma unroll
          for (int k = 0; k < EPV; ++k) acc[v][k] = 0.f;
        }
      }
      load_h<HT>(a.er + (int64_t)j * H, H, erj);
#pragma unroll
      for (int h = 0; h < HT; ++h) dsum[h] = 0.f;
      // candidate out-edges: pass 0: t -> t + o, pass 1: t -> t - o (o = lane + 1 + 32 q), pass 2: self
      const int nself = (cp_w[ti + 1] - cp_w[ti]) - __popcll(lm_w[ti]) - __popcll(rm_w[ti]);
      for (int pass = 0; pass < 3; ++pass) {
        for (int q0 = 0; q0 < (pass == 2 ? 1 : (om + 31) / 32); ++q0) {
          bool ok = false;
          int wi = 0, pos = 0;
          if (pass < 2) {
            const int o = q0 * 32 + lane + 1;
            const int64_t tp = pass == 0 ? t + o : t - o;
            if (o <= om && tp >= wlo && tp < whi) {
              const int di = (int)(tp - wlo);
              const unsigned long long bit = 1ull << (o - 1);
              if (pass == 0 && (lm_w[di] & bit)) {   // source to the left of its destination: an lmask entry
                ok = true;
                pos = cp_w[di] + __popcll(lm_w[di] & (bit - 1));
              } else if (pass == 1 && (rm_w[di] & bit)) {
                ok = true;
                pos = cp_w[di] + __popcll(lm_w[di]) + __popcll(rm_w[di] & (bit - 1));
              }
              wi = di;
            }
          } else if (lane == 0 && nself > 0) {
            ok = true;
            wi = ti;
            pos = cp_w[ti + 1] - 1;
          }
          const unsigned msk = __ballot_sync(FULL, ok);
          if (ok) {
            const int slot = __popc(msk & ((1u << lane) - 1));
            s_wi[w][slot] = wi;
            s_pos[w][slot] = pos;
            s_c[w][slot] = (float)a.B.cnt[pos];
          }
          __syncwarp();
          const int ne = __popc(msk);
          for (int k = 0; k < ne; ++k) {
            const int di = s_wi[w][k];
            const float c = s_c[w][k];
            const uint4 *gr = rows + (size_t)di * V * 32 + lane;
            float p[V], xg[V][EPV];
#pragma unroll
            for (int v = 0; v < V; ++v) {
              unpack(gr[v * 32], xg[v], T());
              float d = 0.f;
#pragma unroll
              for (int kk = 0; kk < EPV; ++kk) d = fmaf(xg[v][kk], whf[v][kk], d);
              p[v] = d;
            }
            // per-head dot over the head's lanes (and vectors)
#pragma unroll
            for (int v = 0; v < V; ++v) {
#pragma unroll
              for (int o = (LPH >= G ? G : LPH) / 2; o > 0; o >>= 1) p[v] += __shfl_xor_sync(FULL, p[v], o);
            }
            if constexpr (LPH > G) {   // a head spans LPH / G vectors of a lane
              constexpr int R = LPH / G;
#pragma unroll
              for (int v = 0; v < V; v += R) {
                float sum = 0.f;
#pragma unroll
                for (int r = 0; r < R; ++r) sum += p[v + r];
#pragma unroll
                for (int r = 0; r < R; ++r) p[v + r] = sum;
              }
            }
            const float *e3 = eld + (size_t)di * 3 * HT;
#pragma unroll
            for (int v = 0; v < V; ++v) {
              const int h = hv[v];
              const float z = e3[h] + sel<HT>(erj, h);
              const float al = fexp(leaky(z, a.slope) - e3[HT + h]);
              const float dz = c * al * (p[v] - e3[2 * HT + h]) * (z > 0.f ? 1.f : a.slope);
              const float ca = c * al;
#pragma unroll
              for (int kk = 0; kk < EPV; kk += 2) ffma2s(acc[v][kk], acc[v][kk + 1], xg[v][kk], xg[v][kk + 1], ca);
              // one lane per head records c dz (and sums it)
              const bool lead = LPH >= G ? (lane == 0 && (v % (LPH >= G ? LPH / G : 1)) == 0) : ((lane % LPH) == 0);
              if (lead) {
                a.dzb[(int64_t)s_pos[w][k] * H + h] = dz;
                dsum[h] += dz;
              }
            }
          }
          __syncwarp();
        }
      }
      float *ap = a.accD + t * a.D + lane * EPV;
#pragma unroll
      for (int v = 0; v < V; ++v)
#pragma unroll
        for (int k = 0; k < EPV; k += 4)
          *reinterpret_cast<float4 *>(ap + v * G * EPV + k) = make_float4(acc[v][k], acc[v][k + 1], acc[v][k + 2], acc[v][k + 3]);
      // derp[t][h]: the per-head sums live in the head's lead lane
#pragma unroll
      for (int h = 0; h < HT; ++h) {
        const int lead_lane = LPH >= G ? 0 : ((h * FF / EPV) % G);
        const float d = __shfl_sync(FULL, dsum[h], lead_lane);
        if (lane == 0) a.derp[t * H + h] = d;
      }
    }
  }
}

// delp[t] = sum of c dz over appearance t's band entries (a8, per appearance)
template <int HT>
__global__ void __launch_bounds__(256) band_del_kernel(const BandArgs a) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < a.B.L * HT; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t t = i / HT;
    const int h = (int)(i % HT);
    float d = 0.f;
    for (int k = a.B.cptr[t]; k < a.B.cptr[t + 1]; ++k) d += a.dzb[(int64_t)k * HT + h];
    a.delp[i] = d;
  }
}

// per node (a8): del, der over its appearances (appearance order), dWh = sum accD + der a_r + del a_l,
// and the per-block partials of da_l = sum del Wh, da_r = sum der Wh (fixed order)
template <typename T, int V, int HT>
__global__ void __launch_bounds__(BW * 32) band_node_kernel(const BandArgs a) {
  constexpr int G = 32, EPV = Tr<T>::EPV, FF = G * V * EPV / HT, H = HT;
  __shared__ double s_red[1024];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  int hv[V];
  float dal[V][EPV], dar[V][EPV], alv[V][EPV], arv[V][EPV];
#pragma unroll
  for (int v = 0; v < V; ++v) {
    hv[v] = ((v * G + lane) * EPV) / FF;
#pragma unroll
    for (int k = 0; k < EPV; ++k) {
      dal[v][k] = dar[v][k] = 0.f;
      alv[v][k] = a.al[(v * G + lane) * EPV + k];
      arv[v][k] = a.ar[(v * G + lane) * EPV + k];
    }
  }
  const T *feat = static_cast<const T *>(a.feat);
  for (int64_t x = (int64_t)blockIdx.x * BW + w; x < a.B.n; x += (int64_t)gridDim.x * BW) {
    const int a0 = a.B.app_ptr[x], a1 = a.B.app_ptr[x + 1];
    float del[HT], der[HT], y[V][EPV];
#pragma unroll
    for (int h = 0; h < HT; ++h) { del[h] = 0.f; der[h] = 0.f; }
#pragma unroll
    for (int v = 0; v < V; ++v)
#pragma unroll
      for (int k = 0; k < EPV; ++k) y[v][k] = 0.f;
    for (int q = a0; q < a1; ++q) {
      const int64_t t = a.B.app_idx[q];
#pragma unroll
      for (int h = 0; h < HT; ++h) { del[h] += a.delp[t * H + h]; der[h] += a.derp[t * H + h]; }
      const float *ap = a.accD + t * a.D + lane * EPV;
#pragma unroll
      for (int v = 0; v < V; ++v)
#pragma unroll
        for (int k = 0; k < EPV; ++k) y[v][k] += ap[v * G * EPV + k];
    }
    for (int h = lane; h < H; h += G) a.der[x * H + h] = sel<HT>(der, h);
    float *orow = a.gfeat + x * a.ldgf + lane * EPV;
    const T *wr = feat + x * a.ldf + lane * EPV;
#pragma unroll
    for (int v = 0; v < V; ++v) {
      const float dl = sel<HT>(del, hv[v]), dr = sel<HT>(der, hv[v]);
      float wh[EPV];
      unpack(ldg16(wr + v * G * EPV), wh, T());
#pragma unroll
      for (int k = 0; k < EPV; ++k) {
        orow[v * G * EPV + k] = y[v][k] + dr * arv[v][k] + dl * alv[v][k];
        dal[v][k] = fmaf(dl, wh[k], dal[v][k]);
        dar[v][k] = fmaf(dr, wh[k], dar[v][k]);
      }
    }
  }
  block_partial<G, V, EPV>(dal, s_red, a.pdal + (int64_t)blockIdx.x * a.D, a.D);
  block_partial<G, V, EPV>(dar, s_red, a.pdar + (int64_t)blockIdx.x * a.D, a.D);
}

__global__ void __launch_bounds__(256) band_param_kernel(const BandArgs a, int nblocks) {
  for (int d = blockIdx.x * blockDim.x + threadIdx.x; d < 2 * a.D; d += gridDim.x * blockDim.x) {
    const double *pp = d < a.D ? a.pdal : a.pdar;
    const int c = d % a.D;
    double s = 0.0;
    for (int b = 0; b < nblocks; ++b) s += pp[(int64_t)b * a.D + c];
    (d < a.D ? a.gal : a.gar)[c] = (float)s;
  }
}

}  // namespace
}  // namespace kern

namespace {
size_t a256(size_t x) { return (x + 255) / 256 * 256; }
constexpr int kBandMaxNodeBlocks = 1024;
struct BandWs { size_t m, l, acc, fwd_total, accD, derp, delp, dzb, pdal, pdar, total; };
BandWs band_ws(int64_t L, int64_t n_cnt, int32_t n_slots, int H, int D) {
  BandWs w;
  const size_t s = (size_t)std::max(1, n_slots), Lz = (size_t)std::max<int64_t>(1, L);
  w.m = 0;
  w.l = a256(s * H * 4);
  w.acc = a256(w.l + s * H * 4);
  w.fwd_total = a256(w.acc + s * (size_t)D * 4);
  // backward (mega_band_gat_bwd): per appearance partials and per band entry c dz
  w.accD = 0;
  w.derp = a256(w.accD + Lz * (size_t)D * 4);
  w.delp = a256(w.derp + Lz * H * 4);
  w.dzb = a256(w.delp + Lz * H * 4);
  w.pdal = a256(w.dzb + (size_t)std::max<int64_t>(1, n_cnt) * H * 4);
  w.pdar = a256(w.pdal + (size_t)kBandMaxNodeBlocks * D * 8);
  w.total = std::max(w.fwd_total, a256(w.pdar + (size_t)kBandMaxNodeBlocks * D * 8));
  return w;
}
}  // namespace
}  // namespace mega

using namespace mega;

extern "C" {

mega_status mega_band_gat_workspace_bytes(const mega_band *band, int heads, int head_dim, mega_dtype dtype,
                                          size_t *ws_bytes) {
  clear_error();
  if (!band || !ws_bytes) return fail(MEGA_ERR_INVALID_ARGUMENT, "null argument");
  mega_band_view v;
  mega_band_view_get(band, &v);
  *ws_bytes = band_ws(v.length, v.cptr ? v.cptr[v.length] : 0, (int32_t)v.num_slots, heads, heads * head_dim).total;
  (void)dtype;
  return MEGA_OK;
}

mega_status mega_band_gat_fwd(const mega_band *band, const void *feat, int64_t ldf, const float *attn_l,
                              const float *attn_r, int heads, int head_dim, mega_dtype dtype, float negative_slope,
                              uint32_t flags, void *out, int64_t ldo, float *ctx, void *ws, size_t ws_bytes,
                              mega_stream_t stream) {
  clear_error();
  NvtxRange nvtx_("mega_band_gat_fwd");
  int bdev = -1, dev = 0;
  const BandDev *Bp = band_dev(band, bdev);
  if (!band) return fail(MEGA_ERR_INVALID_ARGUMENT, "null band");
  if (!Bp) return fail(MEGA_ERR_STATE, "band not bound (mega_band_bind_device)");
  cudaGetDevice(&dev);
  if (bdev != dev) return fail(MEGA_ERR_STATE, "band bound to another device");
  int major = 0;
  cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, dev);
  if (major != 10) return fail(MEGA_ERR_UNSUPPORTED, "libmega.so kernels require an sm_100 (B200) device");
  if (!feat || !attn_l || !attn_r || !out || !ctx || !ws) return fail(MEGA_ERR_INVALID_ARGUMENT, "null pointer");
  if (dtype != MEGA_F32 && dtype != MEGA_BF16) return fail(MEGA_ERR_INVALID_ARGUMENT, "bad dtype");
  if (heads != 1 && heads != 2 && heads != 4 && heads != 8) return fail(MEGA_ERR_UNSUPPORTED, "heads must be 1, 2, 4 or 8");
  const int D = heads * head_dim, esz = dtype == MEGA_BF16 ? 2 : 4, epv = 16 / esz;
  if (head_dim % epv || D % (32 * epv)) return fail(MEGA_ERR_UNSUPPORTED, "band kernel: rows of 32 x V 16-byte vectors");
  const int V = D / (32 * epv);
  if (V != 1 && V != 2 && V != 4) return fail(MEGA_ERR_UNSUPPORTED, "band kernel: 1, 2 or 4 vectors per lane");
  const int lph = head_dim / epv;   // lanes per head must divide a 32-lane row slice
  if (lph > 32 ? (lph % 32 || V % (lph / 32)) : (32 % lph)) return fail(MEGA_ERR_UNSUPPORTED, "band kernel: head_dim");
  if (ldf < D || ldo < D || (ldf * esz) % 16 || (ldo * esz) % 16) return fail(MEGA_ERR_INVALID_ARGUMENT, "bad ld");
  const BandDev &B = *Bp;
  const BandWs w = band_ws(B.L, B.n_cnt, B.n_slots, heads, D);
  if (ws_bytes < w.fwd_total) return fail(MEGA_ERR_OUT_OF_MEMORY, "band workspace too small");
  const size_t row_b = (size_t)D * esz, per_row = row_b + 4 * heads + 4;
  const int win_cap = (int)(kern::BAND_SMEM / per_row);
  const int T = win_cap - 2 * B.omega;
  if (T < 8) return fail(MEGA_ERR_UNSUPPORTED, "band kernel: window + 2 omega rows do not fit in shared memory");
  cudaStream_t st = (cudaStream_t)stream;
  const int64_t plane = B.n * heads;
  mega_status rc;
  if (!(flags & MEGA_FLAG_ELER_IN_CTX)) {
    rc = launch_eler_any(dtype, feat, ldf, B.n, 0, attn_l, attn_r, heads, head_dim, ctx, ctx + plane, st);
    if (rc != MEGA_OK) return rc;
  }
  kern::BandArgs a;
  a.B = B;
  a.feat = feat; a.ldf = ldf; a.el = ctx; a.er = ctx + plane; a.lse = ctx + 2 * plane;
  a.slope = negative_slope; a.out = out; a.ldo = ldo;
  char *wb = static_cast<char *>(ws);
  a.ws_m = reinterpret_cast<float *>(wb + w.m);
  a.ws_l = reinterpret_cast<float *>(wb + w.l);
  a.ws_acc = reinterpret_cast<float *>(wb + w.acc);
  a.D = D; a.T = T; a.win_cap = win_cap;
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const int64_t ntiles = (B.L + T - 1) / T;
  bool ok = false;
  auto go = [&](auto fk, auto mk) {
    cudaFuncSetAttribute(fk, cudaFuncAttributeMaxDynamicSharedMemorySize, kern::BAND_SMEM);
    const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(ntiles, 2 * (int64_t)sms));
    if (B.L > 0) fk<<<grid, kern::BW * 32, kern::BAND_SMEM, st>>>(a);
    if (B.n_merges > 0) {
      const int mg = (int)std::min<int64_t>((B.n_merges + kern::BW - 1) / kern::BW, 8 * (int64_t)sms);
      mk<<<std::max(mg, 1), kern::BW * 32, 0, st>>>(a);
    }
    ok = true;
  };
  auto by_h = [&](auto tag_t, auto v_c) {
    using TT = decltype(tag_t);
    constexpr int VV = decltype(v_c)::value;
    switch (heads) {
      case 1: go(kern::band_fwd_kernel<TT, VV, 1>, kern::band_merge_kernel<TT, VV, 1>); break;
      case 2: go(kern::band_fwd_kernel<TT, VV, 2>, kern::band_merge_kernel<TT, VV, 2>); break;
      case 4: go(kern::band_fwd_kernel<TT, VV, 4>, kern::band_merge_kernel<TT, VV, 4>); break;
      default: go(kern::band_fwd_kernel<TT, VV, 8>, kern::band_merge_kernel<TT, VV, 8>); break;
    }
  };
  auto by_v = [&](auto tag_t) {
    if (V == 1) by_h(tag_t, std::integral_constant<int, 1>());
    else if (V == 2) by_h(tag_t, std::integral_constant<int, 2>());
    else by_h(tag_t, std::integral_constant<int, 4>());
  };
  if (dtype == MEGA_BF16) by_v(__nv_bfloat16());
  else by_v(float());
  if (!ok) return fail(MEGA_ERR_UNSUPPORTED, "band kernel shape");
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? MEGA_OK : fail(MEGA_ERR_CUDA, std::string("band kernels: ") + cudaGetErrorString(e));
}

}  // extern "C"

namespace mega {
namespace {
// shared shape checks of the band entry points -> V (vectors per lane) or -1
int band_shape(int heads, int head_dim, mega_dtype dtype) {
  if (dtype != MEGA_F32 && dtype != MEGA_BF16) return -1;
  if (heads != 1 && heads != 2 && heads != 4 && heads != 8) return -1;
  const int D = heads * head_dim, epv = dtype == MEGA_BF16 ? 8 : 4;
  if (head_dim % epv || D % (32 * epv)) return -1;
  const int V = D / (32 * epv);
  if (V != 1 && V != 2 && V != 4) return -1;
  const int lph = head_dim / epv;
  if (lph > 32 ? (lph % 32 || V % (lph / 32)) : (32 % lph)) return -1;
  return V;
}
}  // namespace
}  // namespace mega

extern "C" {

mega_status mega_band_gat_bwd(const mega_band *band, const void *feat, int64_t ldf, const float *attn_l,
                              const float *attn_r, int heads, int head_dim, mega_dtype dtype, float negative_slope,
                              const void *out, int64_t ldo, const void *grad_out, int64_t ldg, float *ctx,
                              float *grad_feat, int64_t ldgf, float *grad_attn_l, float *grad_attn_r, void *ws,
                              size_t ws_bytes, mega_stream_t stream) {
  clear_error();
  NvtxRange nvtx_("mega_band_gat_bwd");
  int bdev = -1, dev = 0;
  if (!band) return fail(MEGA_ERR_INVALID_ARGUMENT, "null band");
  const BandDev *Bp = band_dev(band, bdev);
  if (!Bp) return fail(MEGA_ERR_STATE, "band not bound (mega_band_bind_device)");
  cudaGetDevice(&dev);
  if (bdev != dev) return fail(MEGA_ERR_STATE, "band bound to another device");
  int major = 0;
  cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, dev);
  if (major != 10) return fail(MEGA_ERR_UNSUPPORTED, "libmega.so kernels require an sm_100 (B200) device");
  if (!feat || !attn_l || !attn_r || !out || !grad_out || !ctx || !grad_feat || !grad_attn_l || !grad_attn_r || !ws)
    return fail(MEGA_ERR_INVALID_ARGUMENT, "null pointer");
  const int V = band_shape(heads, head_dim, dtype);
  if (V < 0) return fail(MEGA_ERR_UNSUPPORTED, "band kernels: rows of 32 x 1/2/4 16-byte vectors, heads 1/2/4/8");
  const int D = heads * head_dim, esz = dtype == MEGA_BF16 ? 2 : 4;
  if (ldf < D || ldo < D || ldg < D || ldgf < D || (ldf * esz) % 16 || (ldo * esz) % 16 || (ldg * esz) % 16 ||
      (ldgf * 4) % 16)
    return fail(MEGA_ERR_INVALID_ARGUMENT, "bad leading dimension");
  const BandDev &B = *Bp;
  const BandWs w = band_ws(B.L, B.n_cnt, B.n_slots, heads, D);
  if (ws_bytes < w.total) return fail(MEGA_ERR_OUT_OF_MEMORY, "band workspace too small");
  // window: g rows + (el, lse, Dlt) + node id + masks + cptr per window entry
  const size_t per_row = (size_t)D * esz + 12 * heads + 4 + 16 + 4;
  const int win_cap = (int)((kern::BAND_SMEM - 64) / per_row);
  const int T = win_cap - 1 - 2 * B.omega;
  if (T < 8) return fail(MEGA_ERR_UNSUPPORTED, "band kernel: window + 2 omega rows do not fit in shared memory");
  cudaStream_t st = (cudaStream_t)stream;
  const int64_t plane = B.n * heads;
  kern::BandArgs a{};
  a.B = B;
  a.feat = feat; a.ldf = ldf; a.el = ctx; a.er = ctx + plane; a.lse = ctx + 2 * plane;
  a.dlt = ctx + 3 * plane; a.der = ctx + 4 * plane;
  a.slope = negative_slope; a.out = const_cast<void *>(out); a.ldo = ldo;
  a.gout = grad_out; a.ldg = ldg; a.al = attn_l; a.ar = attn_r;
  char *wb = static_cast<char *>(ws);
  a.accD = reinterpret_cast<float *>(wb + w.accD);
  a.derp = reinterpret_cast<float *>(wb + w.derp);
  a.delp = reinterpret_cast<float *>(wb + w.delp);
  a.dzb = reinterpret_cast<float *>(wb + w.dzb);
  a.pdal = reinterpret_cast<double *>(wb + w.pdal);
  a.pdar = reinterpret_cast<double *>(wb + w.pdar);
  a.gfeat = grad_feat; a.ldgf = ldgf; a.gal = grad_attn_l; a.gar = grad_attn_r;
  a.D = D; a.T = T; a.win_cap = win_cap;
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const int64_t ntiles = (B.L + T - 1) / T;
  const int node_blocks = (int)std::max<int64_t>(1, std::min<int64_t>((B.n + kern::BW - 1) / kern::BW,
                                                                        std::min(2 * sms, kBandMaxNodeBlocks)));
  bool ok = false;
  auto go = [&](auto dk, auto sk, auto delk, auto nk) {
    dk<<<(int)std::min<int64_t>((B.n + kern::BW - 1) / kern::BW, 8 * (int64_t)sms), kern::BW * 32, 0, st>>>(a);
    cudaFuncSetAttribute(sk, cudaFuncAttributeMaxDynamicSharedMemorySize, kern::BAND_SMEM);
    if (B.L > 0) sk<<<(int)std::max<int64_t>(1, std::min<int64_t>(ntiles, 2 * (int64_t)sms)), kern::BW * 32, kern::BAND_SMEM, st>>>(a);
    delk<<<(int)std::max<int64_t>(1, std::min<int64_t>((B.L * heads + 255) / 256, 8 * (int64_t)sms)), 256, 0, st>>>(a);
    nk<<<node_blocks, kern::BW * 32, 0, st>>>(a);
    kern::band_param_kernel<<<(2 * D + 255) / 256, 256, 0, st>>>(a, node_blocks);
    ok = true;
  };
  auto by_h = [&](auto tag_t, auto v_c) {
    using TT = decltype(tag_t);
    constexpr int VV = decltype(v_c)::value;
    switch (heads) {
      case 1: go(kern::band_dlt_kernel<TT, VV, 1>, kern::band_src_kernel<TT, VV, 1>, kern::band_del_kernel<1>, kern::band_node_kernel<TT, VV, 1>); break;
      case 2: go(kern::band_dlt_kernel<TT, VV, 2>, kern::band_src_kernel<TT, VV, 2>, kern::band_del_kernel<2>, kern::band_node_kernel<TT, VV, 2>); break;
      case 4: go(kern::band_dlt_kernel<TT, VV, 4>, kern::band_src_kernel<TT, VV, 4>, kern::band_del_kernel<4>, kern::band_node_kernel<TT, VV, 4>); break;
      default: go(kern::band_dlt_kernel<TT, VV, 8>, kern::band_src_kernel<TT, VV, 8>, kern::band_del_kernel<8>, kern::band_node_kernel<TT, VV, 8>); break;
    }
  };
  auto by_v = [&](auto tag_t) {
    if (V == 1) by_h(tag_t, std::integral_constant<int, 1>());
    else if (V == 2) by_h(tag_t, std::integral_constant<int, 2>());
    else by_h(tag_t, std::integral_constant<int, 4>());
  };
  if (dtype == MEGA_BF16) by_v(__nv_bfloat16());
  else by_v(float());
  if (!ok) return fail(MEGA_ERR_UNSUPPORTED, "band kernel shape");
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? MEGA_OK : fail(MEGA_ERR_CUDA, std::string("band backward kernels: ") + cudaGetErrorString(e));
}

}  // extern "C"
