// NEXT-3: Graph Transformer edge attention, bf16 storage with fp32
// accumulation — the fast path (Table I; DESIGN.md R-gt).
//   s_e = Q_i.K_j / sqrt(F)   alpha = softmax over In(i)   out_i = sum alpha_e V_j
// Built like the GAT kernels (gat_kernels.cu): a group of G lanes owns a work
// item (a destination row or a <= S-edge segment of one, from the layout's
// items), each lane holds V 16-byte vectors of a row (8 bf16), so a K / V / Q /
// g row is fetched with G*V coalesced 128-bit loads; U rows per operand are in
// flight per step; the per-(edge, head) dot products are reduced across the
// lanes of a head with the transpose butterfly; the online softmax state lives
// in registers, replicated over the lanes of a head.  Split rows / sources write
// partial states to slots merged in fixed order (no atomics).  Backward: a
// destination pass (dQ, and (alpha, ds) per edge at its CSR position) and a
// source pass over the CSC (dK, dV), each gathering two rows per edge.
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>

#include "kern_common.cuh"
#include "mega_internal.h"

namespace mega {
namespace gtb {
using namespace kern;
using T = __nv_bfloat16;
constexpr int EPV = 8;

struct Args {
  DevPart L;
  const T *q, *k, *v;
  int64_t ld;
  int H, F, D;
  float scale;
  T *out;                 // fwd: [rows][ldo] bf16
  const T *outc;          // bwd: the stored forward output
  int64_t ldo;
  float *lse;             // [rows][H] (fwd writes, bwd reads)
  const T *g;             // bwd: grad_out [rows][ldg]
  int64_t ldg;
  float *gq, *gk, *gv;    // fp32 grads
  int64_t ldgr;
  float *alpha, *ds;      // [E_p][H] CSR order
  float *ws_m, *ws_l, *ws_acc;        // fwd slots (fwd_items)
  float *ws_dq;                       // dst-pass slots [fwd slots][D]
  float *ws_dk, *ws_dv;               // src-pass slots [bwd slots][D]
  int *ctr;                           // claim counters (fwd, bwd dst, bwd src) or nullptr: static striding
};

// The GAT kernels' schedule: work items in balanced chunks (DevPart::fchunk / bchunk)
// claimed in layout order from a counter, one chunk ahead; without a counter, chunks gid, gid + W, ...
template <int G> struct ChunkSeq {
  const int32_t *bc;
  int64_t n_ch, ch, ch_next, it_end, stride;
  int *ctr;
  unsigned gmask;
  int gl, rb;
  __device__ int64_t claim(int64_t stat) {
    if (!ctr) return stat;
    int c = 0;
    if (gl == 0) c = atomicAdd(ctr, 1);
    return __shfl_sync(gmask, c, rb);
  }
  __device__ int64_t begin() {
    if (ch >= n_ch) return -1;
    it_end = bc ? __ldg(bc + ch + 1) : ch + 1;
    return bc ? __ldg(bc + ch) : ch;
  }
  __device__ int64_t next(int64_t it) {
    if (++it < it_end) return it;
    ch = ch_next;
    ch_next = claim(ch + stride);
    return begin();
  }
  __device__ int64_t first(const int32_t *chunks, int64_t nchunks, int64_t nitems, int *c, int64_t gid, int64_t W,
                           unsigned m, int l, int r) {
    bc = chunks;
    n_ch = chunks ? nchunks : nitems;
    ctr = c;
    gmask = m;
    gl = l;
    rb = r;
    stride = W;
    ch = claim(gid);
    ch_next = claim(ch + stride);
    it_end = 0;
    return begin();
  }
};

template <int G> __device__ __forceinline__ unsigned group_mask(int grp) {
  return G == 32 ? 0xffffffffu : (((1u << G) - 1u) << (grp * G));
}

// ---- forward ----
template <int G, int V, int HT, int U>
__global__ void __launch_bounds__(TPB) gtb_fwd_kernel(const Args a) {
  constexpr int FF = G * V * EPV / HT, LPH = FF / EPV, GPW = 32 / G;
  (void)LPH;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, gl = lane % G, grp = lane / G;
  const unsigned gmask = group_mask<G>(grp);
  const int H = a.H, F = a.F;
  const int64_t stride = (int64_t)gridDim.x * WPB * GPW;
  int hv[V];
#pragma unroll
  for (int v = 0; v < V; ++v) hv[v] = ((v * G + gl) * EPV) / F;
  ChunkSeq<G> seq;
  for (int64_t it = seq.first(a.L.fchunk, a.L.n_fchunks, a.L.n_fwd_items, a.ctr ? a.ctr + 0 : nullptr,
                              ((int64_t)blockIdx.x * WPB + w) * GPW + grp, stride, gmask, gl, grp * G);
       it >= 0; it = seq.next(it)) {
    const int4 item = a.L.fwd_items[it];
    const int64_t row = a.L.row_begin + item.x;
    float q[V][EPV], acc[V][EPV], m[V], S[V];
#pragma unroll
    for (int v = 0; v < V; ++v) {
      unpack(ldg16(a.q + row * a.ld + (v * G + gl) * EPV), q[v], T());
#pragma unroll
      for (int k = 0; k < EPV; ++k) { q[v][k] *= a.scale; acc[v][k] = 0.f; }
      m[v] = -INFINITY;
      S[v] = 0.f;
    }
    for (int base = item.y; base < item.z; base += U) {
      const int cnt = min(U, item.z - base);
      int64_t j[U];
#pragma unroll
      for (int u = 0; u < U; ++u) j[u] = (int64_t)((uint32_t)__ldg(a.L.src + base + min(u, cnt - 1)) & a.L.id_mask);
      uint4 kr[U][V], vr[U][V];
#pragma unroll
      for (int u = 0; u < U; ++u)
#pragma unroll
        for (int v = 0; v < V; ++v) {
          kr[u][v] = ldg16(a.k + j[u] * a.ld + (v * G + gl) * EPV);
          vr[u][v] = ldg16(a.v + j[u] * a.ld + (v * G + gl) * EPV);
        }
      float p[U][V];
#pragma unroll
      for (int u = 0; u < U; ++u)
#pragma unroll
        for (int v = 0; v < V; ++v) {
          float x[EPV];
          unpack(kr[u][v], x, T());
          float s0 = 0.f, s1 = 0.f;
#pragma unroll
          for (int k = 0; k < EPV; k += 2) ffma2v(s0, s1, x[k], x[k + 1], q[v][k], q[v][k + 1]);
          p[u][v] = s0 + s1;
        }
      head_reduce<G, U, V, FF / EPV>(p, gmask);
#pragma unroll
      for (int v = 0; v < V; ++v) {
        float mx = p[0][v];
#pragma unroll
        for (int u = 1; u < U; ++u)
          if (u < cnt) mx = fmaxf(mx, p[u][v]);
        const float mn = fmaxf(m[v], mx);
        const float c = fexp(m[v] - mn);
        S[v] *= c;
#pragma unroll
        for (int k = 0; k < EPV; ++k) acc[v][k] *= c;
#pragma unroll
        for (int u = 0; u < U; ++u) {
          const float wgt = u < cnt ? fexp(p[u][v] - mn) : 0.f;
          S[v] += wgt;
          float x[EPV];
          unpack(vr[u][v], x, T());
#pragma unroll
          for (int k = 0; k < EPV; k += 2) ffma2s(acc[v][k], acc[v][k + 1], x[k], x[k + 1], wgt);
        }
        m[v] = mn;
      }
    }
    if (item.w < 0) {
      T *orow = a.out + (int64_t)item.x * a.ldo;
#pragma unroll
      for (int v = 0; v < V; ++v) {
        const float inv = S[v] > 0.f ? 1.f / S[v] : 0.f;
        float y[EPV];
#pragma unroll
        for (int k = 0; k < EPV; ++k) y[k] = acc[v][k] * inv;
        st16(orow + (v * G + gl) * EPV, pack(y, T()));
        if (head_lead<G, FF / EPV>(gl, v))
          a.lse[(int64_t)item.x * H + hv[v]] = S[v] > 0.f ? m[v] + flog(S[v]) : -INFINITY;
      }
    } else {
      const int64_t slot = item.w;
#pragma unroll
      for (int v = 0; v < V; ++v) {
        float *pa = a.ws_acc + slot * a.D + (v * G + gl) * EPV;
        *reinterpret_cast<float4 *>(pa) = make_float4(acc[v][0], acc[v][1], acc[v][2], acc[v][3]);
        *reinterpret_cast<float4 *>(pa + 4) = make_float4(acc[v][4], acc[v][5], acc[v][6], acc[v][7]);
        if (head_lead<G, FF / EPV>(gl, v)) {
          a.ws_m[slot * H + hv[v]] = m[v];
          a.ws_l[slot * H + hv[v]] = S[v];
        }
      }
    }
  }
}

// fixed-order merge of split rows: M = max m_k, L = sum l_k e^{m_k - M}, out = sum acc_k e^{m_k - M} / L
__global__ void __launch_bounds__(256) gtb_fwd_merge_kernel(const Args a) {
  const int64_t total = (int64_t)a.L.n_fwd_splits * a.D;
  for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < total; t += (int64_t)gridDim.x * blockDim.x) {
    const int64_t sp = t / a.D;
    const int c = (int)(t % a.D), h = c / a.F;
    const int r = a.L.fwd_splits[3 * sp], s0 = a.L.fwd_splits[3 * sp + 1], ns = a.L.fwd_splits[3 * sp + 2];
    float M = -INFINITY;
    for (int s = 0; s < ns; ++s) M = fmaxf(M, a.ws_m[(int64_t)(s0 + s) * a.H + h]);
    float Ls = 0.f, y = 0.f;
    for (int s = 0; s < ns; ++s) {
      const float f = fexp(a.ws_m[(int64_t)(s0 + s) * a.H + h] - M);
      Ls += a.ws_l[(int64_t)(s0 + s) * a.H + h] * f;
      y = fmaf(f, a.ws_acc[(int64_t)(s0 + s) * a.D + c], y);
    }
    a.out[(int64_t)r * a.ldo + c] = __float2bfloat16_rn(y / Ls);
    if (c % a.F == 0) a.lse[(int64_t)r * a.H + h] = M + flog(Ls);
  }
}

// ---- backward, destination pass: dQ; (alpha, ds) per edge ----
template <int G, int V, int HT, int U>
__global__ void __launch_bounds__(TPB) gtb_bwd_dst_kernel(const Args a) {
  constexpr int FF = G * V * EPV / HT, GPW = 32 / G;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, gl = lane % G, grp = lane / G;
  const unsigned gmask = group_mask<G>(grp);
  const int H = a.H, F = a.F;
  const int64_t stride = (int64_t)gridDim.x * WPB * GPW;
  int hv[V];
#pragma unroll
  for (int v = 0; v < V; ++v) hv[v] = ((v * G + gl) * EPV) / F;
  ChunkSeq<G> seq;
  for (int64_t it = seq.first(a.L.fchunk, a.L.n_fchunks, a.L.n_fwd_items, a.ctr ? a.ctr + 1 : nullptr,
                              ((int64_t)blockIdx.x * WPB + w) * GPW + grp, stride, gmask, gl, grp * G);
       it >= 0; it = seq.next(it)) {
    const int4 item = a.L.fwd_items[it];
    const int64_t lrow = item.x, row = a.L.row_begin + lrow;
    float q[V][EPV], g[V][EPV], dq[V][EPV], dl[1][V], lse[V];
#pragma unroll
    for (int v = 0; v < V; ++v) {
      float o[EPV];
      unpack(ldg16(a.q + row * a.ld + (v * G + gl) * EPV), q[v], T());
      unpack(ldg16(a.g + lrow * a.ldg + (v * G + gl) * EPV), g[v], T());
      unpack(ldg16(a.outc + lrow * a.ldo + (v * G + gl) * EPV), o, T());
      float s = 0.f;
#pragma unroll
      for (int k = 0; k < EPV; ++k) { q[v][k] *= a.scale; dq[v][k] = 0.f; s = fmaf(g[v][k], o[k], s); }
      dl[0][v] = s;
      lse[v] = a.lse[lrow * H + hv[v]];
    }
    head_reduce<G, 1, V, FF / EPV>(dl, gmask);   // Dlt_i = g_i . out_i per head (from the stored out)
    for (int base = item.y; base < item.z; base += U) {
      const int cnt = min(U, item.z - base);
      int64_t j[U];
#pragma unroll
      for (int u = 0; u < U; ++u) j[u] = (int64_t)((uint32_t)__ldg(a.L.src + base + min(u, cnt - 1)) & a.L.id_mask);
      uint4 kr[U][V], vr[U][V];
#pragma unroll
      for (int u = 0; u < U; ++u)
#pragma unroll
        for (int v = 0; v < V; ++v) {
          kr[u][v] = ldg16(a.k + j[u] * a.ld + (v * G + gl) * EPV);
          vr[u][v] = ldg16(a.v + j[u] * a.ld + (v * G + gl) * EPV);
        }
      float s[U][V], d[U][V];
#pragma unroll
      for (int u = 0; u < U; ++u)
#pragma unroll
        for (int v = 0; v < V; ++v) {
          float x[EPV], y[EPV];
          unpack(kr[u][v], x, T());
          unpack(vr[u][v], y, T());
          float s0 = 0.f, s1 = 0.f, d0 = 0.f, d1 = 0.f;
#pragma unroll
          for (int k = 0; k < EPV; k += 2) {
            ffma2v(s0, s1, x[k], x[k + 1], q[v][k], q[v][k + 1]);
            ffma2v(d0, d1, y[k], y[k + 1], g[v][k], g[v][k + 1]);
          }
          s[u][v] = s0 + s1;
          d[u][v] = d0 + d1;
        }
      head_reduce<G, U, V, FF / EPV>(s, gmask);
      head_reduce<G, U, V, FF / EPV>(d, gmask);
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const bool ok = u < cnt;
#pragma unroll
        for (int v = 0; v < V; ++v) {
          const float al = ok ? fexp(s[u][v] - lse[v]) : 0.f;
          const float dsv = al * (d[u][v] - dl[0][v]);
          float x[EPV];
          unpack(kr[u][v], x, T());
#pragma unroll
          for (int k = 0; k < EPV; k += 2) ffma2s(dq[v][k], dq[v][k + 1], x[k], x[k + 1], dsv);
          if (ok && head_lead<G, FF / EPV>(gl, v)) {
            a.alpha[(int64_t)(base + u) * H + hv[v]] = al;
            a.ds[(int64_t)(base + u) * H + hv[v]] = dsv;
          }
        }
      }
    }
    float *dst = item.w < 0 ? a.gq + lrow * a.ldgr : a.ws_dq + (int64_t)item.w * a.D;
    const float sc = item.w < 0 ? a.scale : 1.f;
#pragma unroll
    for (int v = 0; v < V; ++v) {
      float *p = dst + (v * G + gl) * EPV;
      *reinterpret_cast<float4 *>(p) = make_float4(dq[v][0] * sc, dq[v][1] * sc, dq[v][2] * sc, dq[v][3] * sc);
      *reinterpret_cast<float4 *>(p + 4) = make_float4(dq[v][4] * sc, dq[v][5] * sc, dq[v][6] * sc, dq[v][7] * sc);
    }
  }
}

// ---- backward, source pass over the CSC: dK_j = sum ds Q_i / sqrt(F), dV_j = sum alpha g_i ----
template <int G, int V, int HT, int U>
__global__ void __launch_bounds__(TPB) gtb_bwd_src_kernel(const Args a) {
  constexpr int GPW = 32 / G;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, gl = lane % G, grp = lane / G;
  const int H = a.H, F = a.F;
  const int64_t stride = (int64_t)gridDim.x * WPB * GPW;
  int hv[V];
#pragma unroll
  for (int v = 0; v < V; ++v) hv[v] = ((v * G + gl) * EPV) / F;
  ChunkSeq<G> seq;
  for (int64_t it = seq.first(a.L.bchunk, a.L.n_bchunks, a.L.n_bwd_items, a.ctr ? a.ctr + 2 : nullptr,
                              ((int64_t)blockIdx.x * WPB + w) * GPW + grp, stride, group_mask<G>(grp), gl, grp * G);
       it >= 0; it = seq.next(it)) {
    const int4 item = a.L.bwd_items[it];
    const int64_t j = item.x;
    float dk[V][EPV], dv[V][EPV];
#pragma unroll
    for (int v = 0; v < V; ++v)
#pragma unroll
      for (int k = 0; k < EPV; ++k) dk[v][k] = dv[v][k] = 0.f;
    for (int base = item.y; base < item.z; base += U) {
      const int cnt = min(U, item.z - base);
      int64_t r[U], pos[U];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const int c = base + min(u, cnt - 1);
        r[u] = (int64_t)((uint32_t)__ldg(a.L.cdst + c) & a.L.id_mask);
        pos[u] = __ldg(a.L.cpos + c);
      }
      uint4 qr[U][V], gr[U][V];
#pragma unroll
      for (int u = 0; u < U; ++u)
#pragma unroll
        for (int v = 0; v < V; ++v) {
          qr[u][v] = ldg16(a.q + (a.L.row_begin + r[u]) * a.ld + (v * G + gl) * EPV);
          gr[u][v] = ldg16(a.g + r[u] * a.ldg + (v * G + gl) * EPV);
        }
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const bool ok = u < cnt;
#pragma unroll
        for (int v = 0; v < V; ++v) {
          const float al = ok ? __ldg(a.alpha + pos[u] * H + hv[v]) : 0.f;
          const float dsv = ok ? __ldg(a.ds + pos[u] * H + hv[v]) : 0.f;
          float x[EPV], y[EPV];
          unpack(qr[u][v], x, T());
          unpack(gr[u][v], y, T());
#pragma unroll
          for (int k = 0; k < EPV; k += 2) {
            ffma2s(dk[v][k], dk[v][k + 1], x[k], x[k + 1], dsv);
            ffma2s(dv[v][k], dv[v][k + 1], y[k], y[k + 1], al);
          }
        }
      }
    }
    const bool fin = item.w < 0;
    float *pk = fin ? a.gk + j * a.ldgr : a.ws_dk + (int64_t)item.w * a.D;
    float *pv = fin ? a.gv + j * a.ldgr : a.ws_dv + (int64_t)item.w * a.D;
    const float sc = fin ? a.scale : 1.f;
#pragma unroll
    for (int v = 0; v < V; ++v) {
      float *p = pk + (v * G + gl) * EPV, *t = pv + (v * G + gl) * EPV;
      *reinterpret_cast<float4 *>(p) = make_float4(dk[v][0] * sc, dk[v][1] * sc, dk[v][2] * sc, dk[v][3] * sc);
      *reinterpret_cast<float4 *>(p + 4) = make_float4(dk[v][4] * sc, dk[v][5] * sc, dk[v][6] * sc, dk[v][7] * sc);
      *reinterpret_cast<float4 *>(t) = make_float4(dv[v][0], dv[v][1], dv[v][2], dv[v][3]);
      *reinterpret_cast<float4 *>(t + 4) = make_float4(dv[v][4], dv[v][5], dv[v][6], dv[v][7]);
    }
  }
}

// fixed-order sums of split rows (dQ) and split sources (dK, dV)
__global__ void __launch_bounds__(256) gtb_bwd_merge_kernel(const Args a) {
  const int64_t nq = (int64_t)a.L.n_fwd_splits * a.D, nk = (int64_t)a.L.n_bwd_splits * a.D;
  for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < nq + nk; t += (int64_t)gridDim.x * blockDim.x) {
    if (t < nq) {
      const int64_t sp = t / a.D;
      const int c = (int)(t % a.D);
      const int r = a.L.fwd_splits[3 * sp], s0 = a.L.fwd_splits[3 * sp + 1], ns = a.L.fwd_splits[3 * sp + 2];
      float y = 0.f;
      for (int s = 0; s < ns; ++s) y += a.ws_dq[(int64_t)(s0 + s) * a.D + c];
      a.gq[(int64_t)r * a.ldgr + c] = y * a.scale;
    } else {
      const int64_t u = t - nq, sp = u / a.D;
      const int c = (int)(u % a.D);
      const int64_t j = a.L.bwd_splits[3 * sp];
      const int s0 = a.L.bwd_splits[3 * sp + 1], ns = a.L.bwd_splits[3 * sp + 2];
      float yk = 0.f, yv = 0.f;
      for (int s = 0; s < ns; ++s) {
        yk += a.ws_dk[(int64_t)(s0 + s) * a.D + c];
        yv += a.ws_dv[(int64_t)(s0 + s) * a.D + c];
      }
      a.gk[j * a.ldgr + c] = yk * a.scale;
      a.gv[j * a.ldgr + c] = yv;
    }
  }
}

}  // namespace gtb

namespace {
template <int X> using GIC = std::integral_constant<int, X>;
// (G, V) of a bf16 row of nv 16-byte vectors (nv = D / 8)
template <typename Fn> bool gtb_dispatch(int nv, Fn &&fn) {
  switch (nv) {
    case 8: fn(GIC<8>(), GIC<1>()); return true;
    case 16: fn(GIC<16>(), GIC<1>()); return true;
    case 32: fn(GIC<32>(), GIC<1>()); return true;
    case 64: fn(GIC<32>(), GIC<2>()); return true;
    case 128: fn(GIC<32>(), GIC<4>()); return true;
    default: return false;
  }
}
template <typename Fn> void gtb_dispatch_h(int H, Fn &&fn) {
  if (H <= 1) fn(GIC<1>());
  else if (H <= 2) fn(GIC<2>());
  else if (H <= 4) fn(GIC<4>());
  else fn(GIC<8>());
}
int gtb_grid(int64_t groups, int gpw, int sms) {
  const int64_t need = (groups + (int64_t)kern::WPB * gpw - 1) / ((int64_t)kern::WPB * gpw);
  return (int)std::max<int64_t>(1, std::min<int64_t>(need, (int64_t)sms * 2));
}
}  // namespace

// workspace of the bf16 GT path: (alpha, ds) per edge and head, plus the split slots
size_t gtb_workspace_bytes(const Part &P, int H, int D) {
  auto al = [](size_t x) { return (x + 255) / 256 * 256; };
  const size_t e = std::max<size_t>(1, P.src.size());
  const size_t fs = (size_t)std::max(1, P.n_fwd_slots), bs = (size_t)std::max(1, P.n_bwd_slots);
  return 2 * al(e * H * 4) + al(fs * H * 4) * 2 + al(fs * D * 4) * 2 + al(bs * D * 4) * 2 + 256;   // + claim counters
}

mega_status gtb_run(const mega_layout *L, int32_t part, bool bwd, const void *q, const void *k, const void *v,
                    int64_t ld, int heads, int head_dim, void *out, int64_t ldo, float *lse, const void *grad_out,
                    int64_t ldg, float *gq, float *gk, float *gv, int64_t ldgr, void *ws, size_t ws_bytes,
                    cudaStream_t st, int sms) {
  const Part &P = L->parts[part];
  const int D = heads * head_dim;
  if (head_dim % 8 || D % 8) return fail(MEGA_ERR_UNSUPPORTED, "bf16 GT: head_dim a multiple of 8");
  const int nv = D / 8, lph = head_dim / 8;
  if ((lph & (lph - 1)) != 0) return fail(MEGA_ERR_UNSUPPORTED, "bf16 GT: head_dim / 8 a power of two");
  if (ws_bytes < gtb_workspace_bytes(P, heads, D)) return fail(MEGA_ERR_OUT_OF_MEMORY, "GT workspace too small");
  auto al = [](size_t x) { return (x + 255) / 256 * 256; };
  const size_t e = std::max<size_t>(1, P.src.size());
  const size_t fs = (size_t)std::max(1, P.n_fwd_slots), bs = (size_t)std::max(1, P.n_bwd_slots);
  char *w = static_cast<char *>(ws);
  gtb::Args a{};
  a.L = P.dev;
  a.q = static_cast<const gtb::T *>(q); a.k = static_cast<const gtb::T *>(k); a.v = static_cast<const gtb::T *>(v);
  a.ld = ld; a.H = heads; a.F = head_dim; a.D = D; a.scale = 1.f / std::sqrt((float)head_dim);
  a.out = static_cast<gtb::T *>(out); a.outc = static_cast<const gtb::T *>(out); a.ldo = ldo; a.lse = lse;
  a.g = static_cast<const gtb::T *>(grad_out); a.ldg = ldg; a.gq = gq; a.gk = gk; a.gv = gv; a.ldgr = ldgr;
  size_t off = 0;
  a.alpha = reinterpret_cast<float *>(w + off); off += al(e * heads * 4);
  a.ds = reinterpret_cast<float *>(w + off); off += al(e * heads * 4);
  a.ws_m = reinterpret_cast<float *>(w + off); off += al(fs * heads * 4);
  a.ws_l = reinterpret_cast<float *>(w + off); off += al(fs * heads * 4);
  a.ws_acc = reinterpret_cast<float *>(w + off); off += al(fs * D * 4);
  a.ws_dq = reinterpret_cast<float *>(w + off); off += al(fs * D * 4);
  a.ws_dk = reinterpret_cast<float *>(w + off); off += al(bs * D * 4);
  a.ws_dv = reinterpret_cast<float *>(w + off); off += al(bs * D * 4);
  a.ctr = nullptr;
  const int64_t nch = std::max<int64_t>(a.L.fchunk ? a.L.n_fchunks : a.L.n_fwd_items,
                                        a.L.bchunk ? a.L.n_bchunks : a.L.n_bwd_items);
  if (nch >= 16 * 16 * (int64_t)sms) {   // claiming pays with many rounds of chunks (as the GAT kernels)
    a.ctr = reinterpret_cast<int *>(w + off);
    cudaError_t ce = cudaMemsetAsync(a.ctr, 0, 3 * sizeof(int), st);
    if (ce != cudaSuccess) return fail(MEGA_ERR_CUDA, std::string("GT counter reset: ") + cudaGetErrorString(ce));
  }
  mega_status rc = MEGA_OK;
  const bool ok = gtb_dispatch(nv, [&](auto gg, auto vv) {
    constexpr int G = decltype(gg)::value, V = decltype(vv)::value;
    gtb_dispatch_h(heads, [&](auto hh) {
      constexpr int HT = decltype(hh)::value;
      constexpr int U = V >= 2 ? 2 : 4;
      if constexpr ((G * V * 8) % HT == 0 && (G * V * 8 / HT) % 8 == 0) {
        if (!bwd) {
          if (a.L.n_fwd_items > 0)
            gtb::gtb_fwd_kernel<G, V, HT, U><<<gtb_grid(a.L.n_fwd_items, 32 / G, sms), kern::TPB, 0, st>>>(a);
          if (a.L.n_fwd_splits > 0)
            gtb::gtb_fwd_merge_kernel<<<std::max(1, std::min(4 * sms, (int)((a.L.n_fwd_splits * (int64_t)D + 255) / 256))),
                                        256, 0, st>>>(a);
        } else {
          if (a.L.n_fwd_items > 0)
            gtb::gtb_bwd_dst_kernel<G, V, HT, U><<<gtb_grid(a.L.n_fwd_items, 32 / G, sms), kern::TPB, 0, st>>>(a);
          if (a.L.n_bwd_items > 0)
            gtb::gtb_bwd_src_kernel<G, V, HT, U><<<gtb_grid(a.L.n_bwd_items, 32 / G, sms), kern::TPB, 0, st>>>(a);
          const int64_t nm = ((int64_t)a.L.n_fwd_splits + a.L.n_bwd_splits) * D;
          if (nm > 0)
            gtb::gtb_bwd_merge_kernel<<<std::max(1, (int)std::min<int64_t>(4 * sms, (nm + 255) / 256)), 256, 0, st>>>(a);
        }
      } else {
        rc = fail(MEGA_ERR_UNSUPPORTED, "bf16 GT: unsupported head shape");
      }
    });
  });
  if (!ok) return fail(MEGA_ERR_UNSUPPORTED, "bf16 GT: heads*head_dim / 8 must be 8, 16, 32, 64 or 128");
  if (rc != MEGA_OK) return rc;
  cudaError_t ce = cudaGetLastError();
  if (ce != cudaSuccess) return fail(MEGA_ERR_CUDA, std::string("gt bf16 kernels: ") + cudaGetErrorString(ce));
  return MEGA_OK;
}

}  // namespace mega
