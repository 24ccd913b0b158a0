// a3-a8: the GAT attention kernels for sm_100a and their C-ABI entry points.
//
// Memory-bound graph operators: no tensor cores here
// (north_star).  Design:
//   * a "group" of G lanes owns one work item (a destination row, or a
//     segment of one); each lane holds V 16-byte vectors of a feature row, so
//     one source row is fetched with G*V coalesced 128-bit loads;
//   * scores are computed once per (edge, head): in the score phase lane l
//     takes edge base+l for all heads and the group updates the online
//     softmax state with shuffles; the first U source rows of the chunk are
//     requested before the scores are evaluated (their addresses only need
//     the source ids), later batches follow from shared memory;
//   * L2 residency comes from the schedule, not from cache hints: work items
//     are grouped into balanced chunks that the groups claim in layout order
//     (DevPart::fchunk / bchunk, a workspace counter), so the rows gathered
//     concurrently stay within about one round of chunks of the MEGA order
//      and its L2 blocks; gathered rows use plain loads;
//   * rows/sources longer than S edges were split by mega_preprocess into
//     segments whose partial softmax states are merged in fixed order
//     (no atomics anywhere on the value path; the claim counter only hands
//     out work).
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <climits>
#include <cmath>
#include <cstdlib>
#include <mutex>
#include <type_traits>
#include <unordered_map>

#include "mega_internal.h"
#include "kern_common.cuh"

namespace mega {
namespace kern {


// ---- a3+a4+a5: fused score / online edge softmax / aggregation ----
// Per chunk of G edges: lane l scores edge base+l for all heads (online
// softmax state updated with shuffles); source rows stream through two
// register batches of U rows (batch b+1 is requested before batch b is
// accumulated).  Batches are branch-free: the tail of a chunk re-reads its
// last row (an L1 hit) with weight p = 0.
// VAR selects the batch pipeline: 0 = two register batches of U (2U rows in
// flight per lane, 2 CTAs/SM), 1 = one batch of U (3 CTAs/SM), 2 = one batch of 2U.
template <int V, int VAR> struct FwdCfg {
  static constexpr int U0 = V >= 4 ? 1 : (V == 2 ? 4 : 8);
  static constexpr int U = VAR == 2 ? 2 * U0 : U0;
  static constexpr bool DB = VAR == 0;
  static constexpr int MINB = V >= 4 ? 1 : (VAR == 1 ? 3 : 2);
};
template <typename T, int G, int V, int HT, int VAR = 0>
__global__ void __launch_bounds__(TPB, FwdCfg<V, VAR>::MINB) gat_fwd_kernel(const FwdArgs a) {
  constexpr int EPV = Tr<T>::EPV, FF = G * V * EPV / HT, LPH = FF / EPV, GPW = 32 / G, SP = HT + 1;
  constexpr int U = FwdCfg<V, VAR>::U < G ? FwdCfg<V, VAR>::U : G;  // U divides G
  constexpr bool DB = FwdCfg<V, VAR>::DB;
  __shared__ float s_p[WPB][32][SP];
  __shared__ int s_j[WPB][32];  // packed source id (class bits + id)
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, gl = lane % G, grp = lane / G;
  const unsigned gmask = G == 32 ? 0xffffffffu : (((1u << G) - 1u) << (grp * G));
  constexpr int H = HT;   // heads is a power of two <= 8, dispatched as HT == heads (check_shape)
  const int rb = grp * G;
  const uint32_t idm = a.L.id_mask, ldf = (uint32_t)a.ldf;
  const uint64_t pol_cold = policy_first();
  const float *sp_v[V];
#pragma unroll
  for (int v = 0; v < V; ++v) sp_v[v] = &s_p[w][rb][((v * G + gl) * EPV) / FF];
  const T *featl = static_cast<const T *>(a.feat) + gl * EPV;
  const int64_t stride = (int64_t)gridDim.x * WPB * GPW;
  // element offsets fit in 32 bits (checked on the host: n * ldf < 2^32)
  auto row_load = [&](uint4 (&r)[V], uint32_t jj) {
    const T *rp = featl + (jj & idm) * ldf;
#pragma unroll
    for (int v = 0; v < V; ++v) r[v] = ldg16(rp + v * G * EPV);
  };
  for (int64_t it = ((int64_t)blockIdx.x * WPB + w) * GPW + grp; it < a.L.n_fwd_items; it += stride) {
    const int4 item = a.L.fwd_items[it];
    const int64_t grow = a.L.row_begin + item.x;
    float elr[HT], mrun[HT], lrun[HT];
    load_h<HT>(a.el + grow * H, H, elr);
#pragma unroll
    for (int h = 0; h < HT; ++h) { mrun[h] = -INFINITY; lrun[h] = 0.f; }
    float acc[V][EPV];
#pragma unroll
    for (int v = 0; v < V; ++v)
#pragma unroll
      for (int k = 0; k < EPV; ++k) acc[v][k] = 0.f;
    for (int base = item.y; base < item.z; base += G) {
      const int e = base + gl;
      const bool valid = e < item.z;
      const int cnt = min(G, item.z - base), nb = (cnt + U - 1) / U;
      const int jr = ld_stream(a.L.src + min(e, item.z - 1), pol_cold);
      float erj[HT];
      load_h<HT>(a.er + (int64_t)((uint32_t)jr & idm) * H, H, erj);
      uint4 ra[U][V], rz[DB ? U : 1][V];
#pragma unroll
      for (int u = 0; u < U; ++u) row_load(ra[u], (uint32_t)__shfl_sync(gmask, jr, min(u, cnt - 1), G));
      s_j[w][lane] = jr;
      __syncwarp(gmask);
      if (DB && nb > 1) {
#pragma unroll
        for (int u = 0; u < U; ++u) row_load(rz[u], (uint32_t)s_j[w][rb + min(U + u, cnt - 1)]);
      }
      float sc[HT];
#pragma unroll
      for (int h = 0; h < HT; ++h) {
        sc[h] = 1.f;
        if (h < H) {
          const float s = valid ? leaky(elr[h] + erj[h], a.slope) : -INFINITY;
          const float mn = fmaxf(mrun[h], gmax<G>(s, gmask));
          sc[h] = fexp(mrun[h] - mn);
          const float p = valid ? fexp(s - mn) : 0.f;
          lrun[h] = fmaf(lrun[h], sc[h], p);
          mrun[h] = mn;
          s_p[w][lane][h] = p;
        }
      }
#pragma unroll
      for (int v = 0; v < V; ++v) {
        const float f = sel<HT>(sc, ((v * G + gl) * EPV) / FF);
#pragma unroll
        for (int k = 0; k < EPV; ++k) acc[v][k] *= f;
      }
      __syncwarp(gmask);
      auto consume = [&](const uint4 (&raw)[U][V], int k0) {
#pragma unroll
        for (int u = 0; u < U; ++u)
#pragma unroll
          for (int v = 0; v < V; ++v) {
            const float pw = sp_v[v][(k0 + u) * SP];
            float x[EPV];
            unpack(raw[u][v], x, T());
#pragma unroll
            for (int k = 0; k < EPV; k += 2) ffma2s(acc[v][k], acc[v][k + 1], x[k], x[k + 1], pw);
          }
      };
      if constexpr (DB) {
        for (int b = 0; b < nb; b += 2) {
          consume(ra, b * U);
          if (b + 2 < nb) {
#pragma unroll
            for (int u = 0; u < U; ++u) row_load(ra[u], (uint32_t)s_j[w][rb + min((b + 2) * U + u, cnt - 1)]);
          }
          if (b + 1 < nb) {
            consume(rz, (b + 1) * U);
            if (b + 3 < nb) {
#pragma unroll
              for (int u = 0; u < U; ++u) row_load(rz[u], (uint32_t)s_j[w][rb + min((b + 3) * U + u, cnt - 1)]);
            }
          }
        }
      } else {
        for (int b = 0; b < nb; ++b) {
          if (b > 0) {
#pragma unroll
            for (int u = 0; u < U; ++u) row_load(ra[u], (uint32_t)s_j[w][rb + min(b * U + u, cnt - 1)]);
          }
          consume(ra, b * U);
        }
      }
      __syncwarp(gmask);
    }
    float lt[HT];
#pragma unroll
    for (int h = 0; h < HT; ++h) lt[h] = h < H ? gsum<G>(lrun[h], gmask) : 0.f;
    if (item.w < 0) {
      T *orow = static_cast<T *>(a.out) + (int64_t)item.x * a.ldo + gl * EPV;
#pragma unroll
      for (int v = 0; v < V; ++v) {
        const float Lh = sel<HT>(lt, ((v * G + gl) * EPV) / FF);
        const float inv = Lh > 0.f ? 1.f / Lh : 0.f;
        float y[EPV];
#pragma unroll
        for (int k = 0; k < EPV; ++k) y[k] = acc[v][k] * inv;
        st16(orow + v * G * EPV, pack(y, T()));
      }
      for (int h = gl; h < H; h += G) {
        const float Lh = sel<HT>(lt, h);
        a.lse[grow * H + h] = Lh > 0.f ? sel<HT>(mrun, h) + flog(Lh) : -INFINITY;
      }
    } else {
      const int64_t slot = item.w;
      for (int h = gl; h < H; h += G) {
        a.ws_m[slot * H + h] = sel<HT>(mrun, h);
        a.ws_l[slot * H + h] = sel<HT>(lt, h);
      }
      float *pr = a.ws_acc + slot * a.D + gl * EPV;
#pragma unroll
      for (int v = 0; v < V; ++v)
#pragma unroll
        for (int k = 0; k < EPV; k += 4)
          *reinterpret_cast<float4 *>(pr + v * G * EPV + k) =
              make_float4(acc[v][k], acc[v][k + 1], acc[v][k + 2], acc[v][k + 3]);
    }
  }
}

// ---- a3+a4+a5, chunk-pipelined (the default) ----
// The same per-chunk arithmetic as gat_fwd_kernel, but the dependency chain
// item descriptor -> source ids -> er / source rows is taken off the critical
// path: while chunk c is scored and aggregated, the NEXT chunk of the group's
// stream (the next G edges of this item, else the first G of its next item)
// has its source ids, el and er staged in shared memory with cp.async, and its
// source rows prefetched into L2 by the TMA engine (cp.async.bulk.prefetch),
// so chunk c+1 starts with everything but the row bytes on chip and the row
// loads hit L2.  Item descriptors are staged G at a time, double-buffered.
template <typename T, int G, int V, int HT>
__global__ void __launch_bounds__(TPB, FwdCfg<V, 0>::MINB) gat_fwd_pipe_kernel(const FwdArgs a) {
  constexpr int EPV = Tr<T>::EPV, FF = G * V * EPV / HT, GPW = 32 / G, SP = HT + 1;
  constexpr int U = FwdCfg<V, 0>::U < G ? FwdCfg<V, 0>::U : G;  // U divides G
  __shared__ float s_p[WPB][32][SP];
  __shared__ int4 s_desc[2][WPB][32];
  __shared__ int s_src[2][WPB][32];  // packed source ids (class bits + id) of a chunk
  __shared__ __align__(16) float s_er[2][WPB][32][HT];
  __shared__ __align__(16) float s_el[2][WPB][GPW][HT];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, gl = lane % G, grp = lane / G;
  const unsigned gmask = G == 32 ? 0xffffffffu : (((1u << G) - 1u) << (grp * G));
  constexpr int H = HT;   // heads is a power of two <= 8, dispatched as HT == heads (check_shape)
  const int rb = grp * G;
  const uint32_t idm = a.L.id_mask, ldf = (uint32_t)a.ldf;
  const uint64_t pol_st = a.st_hint ? policy_first() : policy_normal();
  const float *sp_v[V];
#pragma unroll
  for (int v = 0; v < V; ++v) sp_v[v] = &s_p[w][rb][((v * G + gl) * EPV) / FF];
  const T *feat = static_cast<const T *>(a.feat);
  const T *featl = feat + gl * EPV;
  // the group's work: a sequence of chunks of the balanced schedule (DevPart::fchunk: items [b, b + n),
  // n <= 8 <= G; without one, the k-GPU passes, one item per chunk), one descriptor batch per chunk.
  // Chunks are claimed in layout order from a counter (a.ctr), three batches ahead of use, so the
  // groups work on a window of about one round of chunks however unevenly the warps are scheduled;
  // a.ctr == nullptr: static striding, chunk gid + k W for the group's batch k (MEGA_SCHED_DYN=0)
  const int64_t W = (int64_t)gridDim.x * WPB * GPW, gid = ((int64_t)blockIdx.x * WPB + w) * GPW + grp;
  const int32_t *fc = a.L.fchunk;
  const int64_t n_ch = fc ? a.L.n_fchunks : a.L.n_fwd_items;
  // rows by element offset: stage_er replaces each staged source id by (id * ldf) once per edge
  auto row_load = [&](uint4 (&r)[V], uint32_t off) {
    const T *rp = featl + off;
#pragma unroll
    for (int v = 0; v < V; ++v) r[v] = ldg16(rp + v * G * EPV);
  };
  auto next_chunk = [&](int k) -> int64_t {
    if (a.ctr) {
      int c = 0;
      if (gl == 0) c = atomicAdd(a.ctr, 1);
      return __shfl_sync(gmask, c, rb);
    }
    return gid + (int64_t)k * W;
  };
  auto bounds = [&](int64_t c, int &b, int &n) {
    b = 0;
    n = 0;
    if (c < n_ch) {
      if (fc) { b = __ldg(fc + c); n = __ldg(fc + c + 1) - b; }
      else { b = (int)c; n = 1; }
    }
  };
  auto stage_desc = [&](int k, int b, int n) {
    if (gl < n) cp_async_small<16>(&s_desc[k & 1][w][rb + gl], a.L.fwd_items + b + gl);
    cp_async_commit();
  };
  // chunk (itm, bse): source ids (tail lanes repeat the last edge) and, for the first chunk of an item, el
  auto stage_src = [&](int b, int4 itm, int bse) {
    if (itm.z > itm.y) cp_async_small<4>(&s_src[b][w][rb + gl], a.L.src + min(bse + gl, itm.z - 1));
    else s_src[b][w][rb + gl] = 0;
    if (bse == itm.y && gl == 0) cp_async_h<HT>(&s_el[b][w][grp][0], a.el + (a.L.row_begin + itm.x) * H);
    cp_async_commit();
  };
  // er of the staged chunk's sources
  auto stage_er = [&](int b, int4 itm, int bse) {
    const uint32_t jj = (uint32_t)s_src[b][w][rb + gl] & idm;
    cp_async_h<HT>(&s_er[b][w][rb + gl][0], a.er + (int64_t)jj * H);
    cp_async_commit();
    s_src[b][w][rb + gl] = (int)(jj * ldf);   // element offset of the row (n * ldf < 2^32, checked on the host)
  };
  // prologue: descriptor batches 0 and 1 staged, batch 2's bounds in registers, batch 3's chunk claimed
  int kb = 0, cnt_cur, cnt_nxt, b2, n2;
  int64_t c3;
  {
    int b0, b1;
    bounds(next_chunk(0), b0, cnt_cur);
    if (cnt_cur == 0) return;
    bounds(next_chunk(1), b1, cnt_nxt);
    stage_desc(0, b0, cnt_cur);
    stage_desc(1, b1, cnt_nxt);
    bounds(next_chunk(2), b2, n2);
    c3 = next_chunk(3);
  }
  cp_async_wait<1>();
  __syncwarp(gmask);
  int q = 0;
  int4 item = s_desc[0][w][rb];
  int base = item.y, buf = 0;
  stage_src(0, item, base);
  cp_async_wait<0>();
  __syncwarp(gmask);
  stage_er(0, item, base);
  cp_async_wait<0>();
  __syncwarp(gmask);
  float elr[HT], mrun[HT], lrun[HT], acc[V][EPV];
  while (true) {
    // ---- the next chunk of this group's stream; stage its ids (and el) ----
    int4 nitem = item;
    int nbase = base + G;
    int nq = q;
    bool has_next = true;
    if (nbase >= item.z) {
      nq = q + 1;
      if (nq < cnt_cur) {
        nitem = s_desc[kb & 1][w][rb + nq];
        nbase = nitem.y;
      } else if (cnt_nxt == 0) {
        has_next = false;
      } else {  // entering descriptor batch kb + 1: make sure it landed, refill the finished buffer
        cp_async_wait<0>();
        __syncwarp(gmask);
        nitem = s_desc[(kb + 1) & 1][w][rb];
        __syncwarp(gmask);
        ++kb;
        nq = 0;
        stage_desc(kb + 1, b2, n2);
        cnt_cur = cnt_nxt;
        cnt_nxt = n2;
        bounds(c3, b2, n2);
        c3 = next_chunk(kb + 3);
        nbase = nitem.y;
      }
    }
    const int nb_ = buf ^ 1;
    if (has_next) stage_src(nb_, nitem, nbase);
    // ---- the current chunk ----
    if (base == item.y) {
#pragma unroll
      for (int h = 0; h < HT; ++h) { elr[h] = s_el[buf][w][grp][h]; mrun[h] = -INFINITY; lrun[h] = 0.f; }
#pragma unroll
      for (int v = 0; v < V; ++v)
#pragma unroll
        for (int k = 0; k < EPV; ++k) acc[v][k] = 0.f;
    }
    const int *sj = &s_src[buf][w][rb];
    const bool valid = base + gl < item.z;
    const int cnt = max(0, min(G, item.z - base)), nbt = (cnt + U - 1) / U;
    uint4 ra[U][V], rz[U][V];
    if (cnt > 0) {
#pragma unroll
      for (int u = 0; u < U; ++u) row_load(ra[u], (uint32_t)sj[min(u, cnt - 1)]);
      if (nbt > 1) {
#pragma unroll
        for (int u = 0; u < U; ++u) row_load(rz[u], (uint32_t)sj[min(U + u, cnt - 1)]);
      }
    }
    float sc[HT];
#pragma unroll
    for (int h = 0; h < HT; ++h) {
      sc[h] = 1.f;
      if (h < H) {
        const float s = valid ? leaky(elr[h] + s_er[buf][w][rb + gl][h], a.slope) : -INFINITY;
        const float mn = fmaxf(mrun[h], gmax<G>(s, gmask));
        sc[h] = mn == -INFINITY ? 1.f : fexp(mrun[h] - mn);
        const float p = valid ? fexp(s - mn) : 0.f;
        lrun[h] = fmaf(lrun[h], sc[h], p);
        mrun[h] = mn;
        s_p[w][lane][h] = p;
      }
    }
    if (base != item.y) {   // acc is 0 in an item's first chunk
#pragma unroll
      for (int v = 0; v < V; ++v) {
        const float f = sel<HT>(sc, ((v * G + gl) * EPV) / FF);
#pragma unroll
        for (int k = 0; k < EPV; ++k) acc[v][k] *= f;
      }
    }
    // next chunk's ids have had the score phase to land: stage its er, prefetch its rows
    cp_async_wait<0>();
    __syncwarp(gmask);
    if (has_next) stage_er(nb_, nitem, nbase);
    auto consume = [&](const uint4 (&raw)[U][V], int k0) {
#pragma unroll
      for (int u = 0; u < U; ++u)
#pragma unroll
        for (int v = 0; v < V; ++v) {
          const float pw = sp_v[v][(k0 + u) * SP];
          float x[EPV];
          unpack(raw[u][v], x, T());
#pragma unroll
          for (int k = 0; k < EPV; k += 2) ffma2s(acc[v][k], acc[v][k + 1], x[k], x[k + 1], pw);
        }
    };
    for (int b = 0; b < nbt; b += 2) {
      consume(ra, b * U);
      if (b + 2 < nbt) {
#pragma unroll
        for (int u = 0; u < U; ++u) row_load(ra[u], (uint32_t)sj[min((b + 2) * U + u, cnt - 1)]);
      }
      if (b + 1 < nbt) {
        consume(rz, (b + 1) * U);
        if (b + 3 < nbt) {
#pragma unroll
          for (int u = 0; u < U; ++u) row_load(rz[u], (uint32_t)sj[min((b + 3) * U + u, cnt - 1)]);
        }
      }
    }
    // ---- end of the item: finalise ----
    if (base + G >= item.z) {
      const int64_t grow = a.L.row_begin + item.x;
      float lt[HT];
#pragma unroll
      for (int h = 0; h < HT; ++h) lt[h] = h < H ? gsum<G>(lrun[h], gmask) : 0.f;
      if (item.w < 0) {
        T *orow = static_cast<T *>(a.out) + (int64_t)item.x * a.ldo + gl * EPV;
#pragma unroll
        for (int v = 0; v < V; ++v) {
          const float Lh = sel<HT>(lt, ((v * G + gl) * EPV) / FF);
          const float inv = Lh > 0.f ? 1.f / Lh : 0.f;
          float y[EPV];
#pragma unroll
          for (int k = 0; k < EPV; ++k) y[k] = acc[v][k] * inv;
          st16_pol(orow + v * G * EPV, pack(y, T()), pol_st);
        }
        for (int h = gl; h < H; h += G) {
          const float Lh = sel<HT>(lt, h);
          a.lse[grow * H + h] = Lh > 0.f ? sel<HT>(mrun, h) + flog(Lh) : -INFINITY;
        }
      } else {
        const int64_t slot = item.w;
        for (int h = gl; h < H; h += G) {
          a.ws_m[slot * H + h] = sel<HT>(mrun, h);
          a.ws_l[slot * H + h] = sel<HT>(lt, h);
        }
        float *pr = a.ws_acc + slot * a.D + gl * EPV;
#pragma unroll
        for (int v = 0; v < V; ++v)
#pragma unroll
          for (int k = 0; k < EPV; k += 4)
            *reinterpret_cast<float4 *>(pr + v * G * EPV + k) =
                make_float4(acc[v][k], acc[v][k + 1], acc[v][k + 2], acc[v][k + 3]);
      }
    }
    if (!has_next) break;
    cp_async_wait<0>();
    __syncwarp(gmask);
    item = nitem;
    base = nbase;
    q = nq;
    buf = nb_;
  }
  cp_async_wait<0>();
}

// Merge the partial softmax states of split rows: M = max m_k,
// L = sum l_k e^{m_k - M}, out = sum acc_k e^{m_k - M} / L, lse = M + log L.
template <typename T, int G, int V>
__global__ void __launch_bounds__(TPB) gat_fwd_merge_kernel(const FwdArgs a) {
  constexpr int EPV = Tr<T>::EPV, GPW = 32 / G;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, gl = lane % G, grp = lane / G;
  const int H = a.H;
  const int64_t stride = (int64_t)gridDim.x * WPB * GPW;
  for (int64_t it = ((int64_t)blockIdx.x * WPB + w) * GPW + grp; it < a.L.n_fwd_splits; it += stride) {
    const int r = a.L.fwd_splits[3 * it], s0 = a.L.fwd_splits[3 * it + 1], ns = a.L.fwd_splits[3 * it + 2];
    const int64_t grow = a.L.row_begin + r;
    for (int h = gl; h < H; h += G) {
      float M = -INFINITY;
      for (int k = 0; k < ns; ++k) M = fmaxf(M, a.ws_m[(int64_t)(s0 + k) * H + h]);
      float Ls = 0.f;
      for (int k = 0; k < ns; ++k) Ls += a.ws_l[(int64_t)(s0 + k) * H + h] * fexp(a.ws_m[(int64_t)(s0 + k) * H + h] - M);
      a.lse[grow * H + h] = M + flog(Ls);
    }
    T *orow = static_cast<T *>(a.out) + (int64_t)r * a.ldo;
#pragma unroll
    for (int v = 0; v < V; ++v) {
      const int col = (v * G + gl) * EPV, h = col / a.F;
      float M = -INFINITY;
      for (int k = 0; k < ns; ++k) M = fmaxf(M, a.ws_m[(int64_t)(s0 + k) * H + h]);
      float Ls = 0.f, y[EPV];
#pragma unroll
      for (int q = 0; q < EPV; ++q) y[q] = 0.f;
      for (int k = 0; k < ns; ++k) {
        const float f = fexp(a.ws_m[(int64_t)(s0 + k) * H + h] - M);
        Ls += a.ws_l[(int64_t)(s0 + k) * H + h] * f;
        const float *pa = a.ws_acc + (int64_t)(s0 + k) * a.D + col;
#pragma unroll
        for (int q = 0; q < EPV; ++q) y[q] = fmaf(f, pa[q], y[q]);
      }
      const float inv = 1.f / Ls;
#pragma unroll
      for (int q = 0; q < EPV; ++q) y[q] *= inv;
      st16(orow + col, pack(y, T()));
    }
  }
}

// ---- a2 epilogue (when features did not come from mega_project_fwd): el, er ----
template <typename T, int G, int V, int HT>
__global__ void __launch_bounds__(TPB) eler_kernel(const T *feat, int64_t ldf, int64_t rows, int64_t row0,
                                                   const float *al, const float *ar, int H, int F, float *el,
                                                   float *er) {
  constexpr int EPV = Tr<T>::EPV, GPW = 32 / G, FF = G * V * EPV / HT, LPH = FF / EPV;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, gl = lane % G, grp = lane / G;
  const unsigned gmask = G == 32 ? 0xffffffffu : (((1u << G) - 1u) << (grp * G));
  float cl[V][EPV], cr[V][EPV];
  int hv[V];
#pragma unroll
  for (int v = 0; v < V; ++v) {
    const int col = (v * G + gl) * EPV;
    hv[v] = col / FF;
#pragma unroll
    for (int k = 0; k < EPV; ++k) { cl[v][k] = al[col + k]; cr[v][k] = ar[col + k]; }
  }
  const int64_t stride = (int64_t)gridDim.x * WPB * GPW;
  for (int64_t r = ((int64_t)blockIdx.x * WPB + w) * GPW + grp; r < rows; r += stride) {
    float pl[1][V], pr[1][V];
    const T *rp = feat + r * ldf + gl * EPV;
#pragma unroll
    for (int v = 0; v < V; ++v) {
      float x[EPV];
      unpack(ldg16(rp + v * G * EPV), x, T());
      float sl = 0.f, sr = 0.f;
#pragma unroll
      for (int k = 0; k < EPV; ++k) { sl = fmaf(cl[v][k], x[k], sl); sr = fmaf(cr[v][k], x[k], sr); }
      pl[0][v] = sl; pr[0][v] = sr;
    }
    head_reduce<G, 1, V, LPH>(pl, gmask);
    head_reduce<G, 1, V, LPH>(pr, gmask);
#pragma unroll
    for (int v = 0; v < V; ++v)
      if (head_lead<G, LPH>(gl, v)) {
        el[(row0 + r) * H + hv[v]] = pl[0][v];
        er[(row0 + r) * H + hv[v]] = pr[0][v];
      }
  }
}


// ---- a6: Dlt_i = g_i . out_i ----
template <typename T, int G, int V, int HT>
__global__ void __launch_bounds__(TPB) dlt_kernel(const BwdArgs a) {
  constexpr int EPV = Tr<T>::EPV, GPW = 32 / G, FF = G * V * EPV / HT, LPH = FF / EPV;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, gl = lane % G, grp = lane / G;
  const unsigned gmask = G == 32 ? 0xffffffffu : (((1u << G) - 1u) << (grp * G));
  constexpr int H = HT;   // heads is a power of two <= 8, dispatched as HT == heads (check_shape)
  const int64_t stride = (int64_t)gridDim.x * WPB * GPW;
  for (int64_t r = ((int64_t)blockIdx.x * WPB + w) * GPW + grp; r < a.L.rows; r += stride) {
    const T *gr = static_cast<const T *>(a.gout) + r * a.ldg + gl * EPV;
    const T *orr = static_cast<const T *>(a.out) + r * a.ldo + gl * EPV;
    float p[1][V];
#pragma unroll
    for (int v = 0; v < V; ++v) {
      float x[EPV], y[EPV];
      unpack(ldg16(gr + v * G * EPV), x, T());
      unpack(ldg16(orr + v * G * EPV), y, T());
      float s = 0.f;
#pragma unroll
      for (int k = 0; k < EPV; ++k) s = fmaf(x[k], y[k], s);
      p[0][v] = s;
    }
    head_reduce<G, 1, V, LPH>(p, gmask);
#pragma unroll
    for (int v = 0; v < V; ++v)
      if (head_lead<G, LPH>(gl, v)) a.dlt[(a.L.row_begin + r) * H + ((v * G + gl) * EPV) / FF] = p[0][v];
  }
}

// ---- a7: source-major pass over the CSC ----
// For source j and out-edge (j -> i): alpha = exp(LeakyReLU(el_i + er_j) - lse_i),
// dalpha = g_i . Wh_j, dz = alpha (dalpha - Dlt_i) (z > 0 ? 1 : slope);
// dWh_j = sum alpha g_i + der_j a_r with der_j = sum dz; dz stored at the edge's CSR position,
// der_j into the der plane of ctx.  g rows stream through two register
// batches; batches are branch-free (the chunk tail re-reads its last row with
// alpha = 0).
// VAR: 0 = two register batches of U rows, 1 = one batch of 2U rows.
template <typename T, int G, int V, int HT, int VAR = 0>
__global__ void __launch_bounds__(TPB, (V >= 4 ? 1 : 2)) gat_bwd_src_kernel(const BwdArgs a) {
  constexpr int EPV = Tr<T>::EPV, FF = G * V * EPV / HT, LPH = FF / EPV, GPW = 32 / G, SP = HT + 1;
  constexpr int U1 = V >= 4 ? 1 : (V == 2 ? 2 : 4), U0 = VAR == 1 ? 2 * U1 : U1, U = U0 < G ? U0 : G;
  constexpr bool DB = VAR == 0;
  // transpose-butterfly reduction of the U*V per-lane dot products over the
  // LPH lanes of a head: log2(LPH) shuffles per batch instead of U*V*log2(LPH),
  // and each lane then owns one (edge, vector) value (index `bidx`)
  constexpr int NB = U * V;
  constexpr bool BFLY = LPH >= 2 && LPH <= G && NB >= 2 && NB <= LPH;
  constexpr int UB = U == 1 ? 0 : (U == 2 ? 1 : (U == 4 ? 2 : 3));
  __shared__ float s_a[WPB][32][SP];  // alpha, sign bit = (z <= 0)
  __shared__ float s_d[WPB][32][SP];  // Dlt_i
  __shared__ float s_z[WPB][32][SP];  // dz out
  __shared__ int s_i[WPB][32];        // packed destination row
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, gl = lane % G, grp = lane / G;
  const unsigned gmask = G == 32 ? 0xffffffffu : (((1u << G) - 1u) << (grp * G));
  constexpr int H = HT;   // heads is a power of two <= 8, dispatched as HT == heads (check_shape)
  const int rb = grp * G;
  const uint32_t idm = a.L.id_mask, ldg = (uint32_t)a.ldg;
  const uint64_t pol_cold = policy_first();
  int hv[V];
#pragma unroll
  for (int v = 0; v < V; ++v) hv[v] = ((v * G + gl) * EPV) / FF;
  int bidx = 0;  // butterfly: the (u, v) value this lane ends up holding, i = u * V + v
#pragma unroll
  for (int s = 0, o = LPH >> 1; (1 << s) < NB; ++s, o >>= 1) bidx = 2 * bidx + ((gl & o) ? 1 : 0);
  const int bu = bidx / V, bv = bidx % V;
  const int bhead = ((bv * G + gl) * EPV) / FF;
  const bool bwriter = (gl & (LPH / (NB > 0 ? NB : 1) - 1)) == 0;
  const T *feat = static_cast<const T *>(a.feat);
  const T *goutl = static_cast<const T *>(a.gout) + gl * EPV;
  const int64_t stride = (int64_t)gridDim.x * WPB * GPW;
  auto row_load = [&](uint4 (&r)[V], uint32_t ii) {
    const T *rp = goutl + (ii & idm) * ldg;
#pragma unroll
    for (int v = 0; v < V; ++v) r[v] = ldg16(rp + v * G * EPV);
  };
  for (int64_t it = ((int64_t)blockIdx.x * WPB + w) * GPW + grp; it < a.L.n_bwd_items; it += stride) {
    const int4 item = a.L.bwd_items[it];
    const int64_t j = item.x;
    float whf[V][EPV], acc[V][EPV], derv[V], dacc = 0.f;
    {
      const T *rp = feat + j * a.ldf + gl * EPV;
#pragma unroll
      for (int v = 0; v < V; ++v) {
        unpack(ldg16(rp + v * G * EPV), whf[v], T());
        derv[v] = 0.f;
#pragma unroll
        for (int k = 0; k < EPV; ++k) acc[v][k] = 0.f;
      }
    }
    float erj[HT];
    load_h<HT>(a.er + j * H, H, erj);
    for (int base = item.y; base < item.z; base += G) {
      const int c = base + gl;
      const bool valid = c < item.z;
      const int cp_c = ld_stream(a.L.cpos + min(c, item.z - 1), policy_first());  // dz's CSR position
      const int cnt = min(G, item.z - base), nb = (cnt + U - 1) / U;
      const int ir = ld_stream(a.L.cdst + min(c, item.z - 1), pol_cold);
      const int64_t gi = a.L.row_begin + (int)((uint32_t)ir & idm);
      float eli[HT], lsei[HT], dli[HT];
      load_h<HT>(a.el + gi * H, H, eli);
      load_h<HT>(a.lse + gi * H, H, lsei);
      load_h<HT>(a.dlt + gi * H, H, dli);
      uint4 ra[U][V], rz[DB ? U : 1][V];
#pragma unroll
      for (int u = 0; u < U; ++u) row_load(ra[u], (uint32_t)__shfl_sync(gmask, ir, min(u, cnt - 1), G));
      s_i[w][lane] = ir;
      __syncwarp(gmask);
      if (DB && nb > 1) {
#pragma unroll
        for (int u = 0; u < U; ++u) row_load(rz[u], (uint32_t)s_i[w][rb + min(U + u, cnt - 1)]);
      }
#pragma unroll
      for (int h = 0; h < HT; ++h)
        if (h < H) {
          const float z = eli[h] + erj[h];
          const float al = valid ? fexp(leaky(z, a.slope) - lsei[h]) : 0.f;
          s_a[w][lane][h] = z > 0.f ? al : -al;
          s_d[w][lane][h] = dli[h];
        }
      __syncwarp(gmask);
      auto consume = [&](const uint4 (&raw)[U][V], int k0) {
        float p[U][V];
#pragma unroll
        for (int u = 0; u < U; ++u)
#pragma unroll
          for (int v = 0; v < V; ++v) {
            // alpha is known before the dot product: accumulate alpha g_i and g_i . Wh_j in one pass
            const float al = fabsf(s_a[w][rb + k0 + u][hv[v]]);
            float x[EPV];
            unpack(raw[u][v], x, T());
            float s0 = 0.f, s1 = 0.f;
#pragma unroll
            for (int k = 0; k < EPV; k += 2) {
              ffma2v(s0, s1, x[k], x[k + 1], whf[v][k], whf[v][k + 1]);
              ffma2s(acc[v][k], acc[v][k + 1], x[k], x[k + 1], al);
            }
            p[u][v] = s0 + s1;
          }
        if constexpr (BFLY) {
          float q[NB];
#pragma unroll
          for (int i = 0; i < NB; ++i) q[i] = p[i / V][i % V];
#pragma unroll
          for (int n = NB, o = LPH >> 1; o > 0; o >>= 1) {
            if (n > 1) {
              const bool up = (gl & o) != 0;
#pragma unroll
              for (int i = 0; i < n / 2; ++i) {
                const float send = up ? q[i] : q[i + n / 2];
                const float keep = up ? q[i + n / 2] : q[i];
                q[i] = keep + __shfl_xor_sync(gmask, send, o, G);
              }
              n /= 2;
            } else {
              q[0] += __shfl_xor_sync(gmask, q[0], o, G);
            }
          }
          const int er_ = rb + k0 + bu;
          const float sa = s_a[w][er_][bhead];
          const float dz = fabsf(sa) * (q[0] - s_d[w][er_][bhead]) * (signbit(sa) ? a.slope : 1.f);
          dacc += dz;
          if (bwriter) s_z[w][er_][bhead] = dz;
        } else {
          head_reduce<G, U, V, LPH>(p, gmask);
#pragma unroll
          for (int u = 0; u < U; ++u) {
            const int er_ = rb + k0 + u;
#pragma unroll
            for (int v = 0; v < V; ++v) {
              const float sa = s_a[w][er_][hv[v]];
              const float dz = fabsf(sa) * (p[u][v] - s_d[w][er_][hv[v]]) * (signbit(sa) ? a.slope : 1.f);
              derv[v] += dz;
              if (head_lead<G, LPH>(gl, v)) s_z[w][er_][hv[v]] = dz;
            }
          }
        }
      };
      if constexpr (DB) {
        for (int b = 0; b < nb; b += 2) {
          consume(ra, b * U);
          if (b + 2 < nb) {
#pragma unroll
            for (int u = 0; u < U; ++u) row_load(ra[u], (uint32_t)s_i[w][rb + min((b + 2) * U + u, cnt - 1)]);
          }
          if (b + 1 < nb) {
            consume(rz, (b + 1) * U);
            if (b + 3 < nb) {
#pragma unroll
              for (int u = 0; u < U; ++u) row_load(rz[u], (uint32_t)s_i[w][rb + min((b + 3) * U + u, cnt - 1)]);
            }
          }
        }
      } else {
        for (int b = 0; b < nb; ++b) {
          if (b > 0) {
#pragma unroll
            for (int u = 0; u < U; ++u) row_load(ra[u], (uint32_t)s_i[w][rb + min(b * U + u, cnt - 1)]);
          }
          consume(ra, b * U);
        }
      }
      __syncwarp(gmask);
      if (valid) {
        float *dzp = a.dz + (int64_t)cp_c * H;  // CSR order
        if (HT >= 4 && (H & 3) == 0) {
#pragma unroll
          for (int q = 0; q < HT / 4; ++q)
            if (4 * q < H)
              reinterpret_cast<float4 *>(dzp)[q] = make_float4(s_z[w][lane][4 * q], s_z[w][lane][4 * q + 1],
                                                               s_z[w][lane][4 * q + 2], s_z[w][lane][4 * q + 3]);
        } else {
          for (int h = 0; h < H; ++h) dzp[h] = s_z[w][lane][h];
        }
      }
      __syncwarp(gmask);
    }
    if constexpr (BFLY) {  // sum over the edge slots u, then fetch each vector's head total
      float dsum = dacc;
#pragma unroll
      for (int s = 0, o = LPH >> 1; s < UB; ++s, o >>= 1) dsum += __shfl_xor_sync(gmask, dsum, o, G);
#pragma unroll
      for (int v = 0; v < V; ++v) {
        int src = gl;
#pragma unroll
        for (int t = 0, o = LPH >> (1 + UB); (1 << t) < V; ++t, o >>= 1) {
          const int bit = (v >> ((V == 2 ? 1 : (V == 4 ? 2 : 3)) - 1 - t)) & 1;
          src = bit ? (src | o) : (src & ~o);
        }
        derv[v] = __shfl_sync(gmask, dsum, src, G);
      }
    }
    if (item.w < 0) {
      float *orow = a.gfeat + j * a.ldgf + gl * EPV;
#pragma unroll
      for (int v = 0; v < V; ++v) {
        const float *arp = a.ar + (v * G + gl) * EPV;
        float y[EPV];
#pragma unroll
        for (int k = 0; k < EPV; k += 4) {
          const float4 r4 = __ldg(reinterpret_cast<const float4 *>(arp + k));
          y[k] = fmaf(derv[v], r4.x, acc[v][k]); y[k + 1] = fmaf(derv[v], r4.y, acc[v][k + 1]);
          y[k + 2] = fmaf(derv[v], r4.z, acc[v][k + 2]); y[k + 3] = fmaf(derv[v], r4.w, acc[v][k + 3]);
          if (!a.lp_partial)
            *reinterpret_cast<float4 *>(orow + v * G * EPV + k) = make_float4(y[k], y[k + 1], y[k + 2], y[k + 3]);
        }
        if (a.lp_partial) st16(static_cast<T *>(a.gfeat_lp) + j * a.ldlp + (v * G + gl) * EPV, pack(y, T()));
        if (head_lead<G, LPH>(gl, v)) a.der[j * H + hv[v]] = derv[v];
      }
    } else {
      const int64_t slot = item.w;
      float *pr = a.ws_bacc + slot * a.D + gl * EPV;
#pragma unroll
      for (int v = 0; v < V; ++v) {
#pragma unroll
        for (int k = 0; k < EPV; k += 4)
          *reinterpret_cast<float4 *>(pr + v * G * EPV + k) =
              make_float4(acc[v][k], acc[v][k + 1], acc[v][k + 2], acc[v][k + 3]);
        if (head_lead<G, LPH>(gl, v)) a.ws_bder[slot * H + hv[v]] = derv[v];
      }
    }
  }
}

// ---- a7 with a shared-memory ring (G = 32) ----
// gat_bwd_src_kernel's arithmetic, but the g rows of a chunk stream through a
// per-warp ring of NBF batches of U rows filled with cp.async (LDGSTS): every
// lane copies and later reads back exactly its own 16-byte pieces, so the ring
// needs no barriers, and NBF*U rows per warp are in flight without holding
// registers (the register-batch kernel keeps 2U = 4 in 125 registers).
template <typename T, int V, int HT, int U, int NBF>
__global__ void __launch_bounds__(TPB, 2) gat_bwd_src_ring_kernel(const BwdArgs a) {
  constexpr int G = 32, EPV = Tr<T>::EPV, FF = G * V * EPV / HT, LPH = FF / EPV, SP = HT + 1;
  constexpr int RS = NBF * U;  // ring slots (U rows per batch)
  constexpr int NB = U * V;
  constexpr bool BFLY = LPH >= 2 && LPH <= G && NB >= 2 && NB <= LPH;
  constexpr int UB = U == 1 ? 0 : (U == 2 ? 1 : (U == 4 ? 2 : 3));
  extern __shared__ uint4 ring_all[];  // [WPB][RS][V][32]
  __shared__ float s_a[WPB][32][SP];
  __shared__ float s_d[WPB][32][SP];
  __shared__ float s_z[WPB][32][SP];
  __shared__ int s_i[WPB][32];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, gl = lane;
  const unsigned gmask = 0xffffffffu;
  constexpr int H = HT;   // heads is a power of two <= 8, dispatched as HT == heads (check_shape)
  uint4 *ring = ring_all + (size_t)w * RS * V * 32;
  const uint32_t idm = a.L.id_mask, ldg = (uint32_t)a.ldg;
  const uint64_t pol_cold = policy_first();
  const uint64_t pol_st = a.st_hint ? policy_first() : policy_normal();
  int hv[V];
#pragma unroll
  for (int v = 0; v < V; ++v) hv[v] = ((v * G + gl) * EPV) / FF;
  int bidx = 0;
#pragma unroll
  for (int s = 0, o = LPH >> 1; (1 << s) < NB; ++s, o >>= 1) bidx = 2 * bidx + ((gl & o) ? 1 : 0);
  const int bu = bidx / V, bv = bidx % V;
  const int bhead = ((bv * G + gl) * EPV) / FF;
  const bool bwriter = (gl & (LPH / (NB > 0 ? NB : 1) - 1)) == 0;
  const T *feat = static_cast<const T *>(a.feat);
  const T *goutl = static_cast<const T *>(a.gout) + gl * EPV;
  const int64_t stride = (int64_t)gridDim.x * WPB;
  // batch b of the chunk (rows bU .. bU+U-1, clamped to the last) -> ring slots (b % NBF) U ..; one group per batch
  auto issue = [&](int b, int cnt) {
    if (b * U < cnt) {
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const T *rp = goutl + (uint32_t)s_i[w][min(b * U + u, cnt - 1)];   // element offset (see below)
        uint4 *dst = ring + (((b % NBF) * U + u) * V) * 32 + lane;
#pragma unroll
        for (int v = 0; v < V; ++v) cp_async16_plain(dst + v * 32, rp + v * G * EPV);
      }
    }
    cp_async_commit();
  };
  // work: chunks c = warp, warp + W, ... of the balanced schedule (DevPart::bchunk; without one,
  // the k-GPU passes over their own item ranges, one item per chunk)
  // chunks are claimed in layout order from a.ctr one chunk ahead of use (as in the forward);
  // a.ctr == nullptr: static striding
  const int32_t *bc = a.L.bchunk;
  const int64_t n_bch = bc ? a.L.n_bchunks : a.L.n_bwd_items;
  auto claim = [&](int64_t stat) -> int64_t {
    if (!a.ctr) return stat;
    int c = 0;
    if (lane == 0) c = atomicAdd(a.ctr, 1);
    return __shfl_sync(gmask, c, 0);
  };
  int64_t ch = claim((int64_t)blockIdx.x * WPB + w), it_end = 0;
  int64_t ch_next = claim(ch + stride);
  auto chunk_begin = [&]() -> int64_t {
    if (ch >= n_bch) return -1;
    it_end = bc ? __ldg(bc + ch + 1) : ch + 1;
    return bc ? __ldg(bc + ch) : ch;
  };
  auto next_item = [&](int64_t it) -> int64_t {
    if (++it < it_end) return it;
    ch = ch_next;
    ch_next = claim(ch + stride);
    return chunk_begin();
  };
  for (int64_t it = chunk_begin(); it >= 0; it = next_item(it)) {
    const int4 item = a.L.bwd_items[it];
    const int64_t j = item.x;
    float whf[V][EPV], acc[V][EPV], derv[V], dacc = 0.f;
    {
      const T *rp = feat + j * a.ldf + gl * EPV;
#pragma unroll
      for (int v = 0; v < V; ++v) {
        unpack(ldg16_pol(rp + v * G * EPV, pol_st), whf[v], T());
        derv[v] = 0.f;
#pragma unroll
        for (int k = 0; k < EPV; ++k) acc[v][k] = 0.f;
      }
    }
    float erj[HT];
    load_h<HT>(a.er + j * H, H, erj);
    for (int base = item.y; base < item.z; base += G) {
      const int c = base + gl;
      const bool valid = c < item.z;
      const int cp_c = ld_stream(a.L.cpos + min(c, item.z - 1), policy_first());  // dz's CSR position
      const int cnt = min(G, item.z - base), nb = (cnt + U - 1) / U;
      const int ir = ld_stream(a.L.cdst + min(c, item.z - 1), pol_cold);
      const int64_t gi = a.L.row_begin + (int)((uint32_t)ir & idm);
      float eli[HT], lsei[HT], dli[HT];
      load_h<HT>(a.el + gi * H, H, eli);
      load_h<HT>(a.lse + gi * H, H, lsei);
      load_h<HT>(a.dlt + gi * H, H, dli);
      s_i[w][lane] = (int)(((uint32_t)ir & idm) * ldg);   // the g row's element offset (n * ldg < 2^32)
      __syncwarp();
#pragma unroll
      for (int b = 0; b < NBF; ++b) issue(b, cnt);
#pragma unroll
      for (int h = 0; h < HT; ++h)
        if (h < H) {
          const float z = eli[h] + erj[h];
          const float al = valid ? fexp(leaky(z, a.slope) - lsei[h]) : 0.f;
          s_a[w][lane][h] = z > 0.f ? al : -al;
          s_d[w][lane][h] = dli[h];
        }
      __syncwarp();
      for (int b = 0; b < nb; ++b) {
        cp_async_wait<NBF - 1>();
        const uint4 *slot = ring + ((b % NBF) * U * V) * 32 + lane;
        const int k0 = b * U;
        float p[U][V];
#pragma unroll
        for (int u = 0; u < U; ++u)
#pragma unroll
          for (int v = 0; v < V; ++v) {
            const float al = fabsf(s_a[w][k0 + u][hv[v]]);
            float x[EPV];
            unpack(slot[(u * V + v) * 32], x, T());
            float s0 = 0.f, s1 = 0.f;
#pragma unroll
            for (int k = 0; k < EPV; k += 2) {
              ffma2v(s0, s1, x[k], x[k + 1], whf[v][k], whf[v][k + 1]);
              ffma2s(acc[v][k], acc[v][k + 1], x[k], x[k + 1], al);
            }
            p[u][v] = s0 + s1;
          }
        issue(b + NBF, cnt);  // refill the slot just read (this lane's own pieces)
        if constexpr (BFLY) {
          float q[NB];
#pragma unroll
          for (int i = 0; i < NB; ++i) q[i] = p[i / V][i % V];
#pragma unroll
          for (int n = NB, o = LPH >> 1; o > 0; o >>= 1) {
            if (n > 1) {
              const bool up = (gl & o) != 0;
#pragma unroll
              for (int i = 0; i < n / 2; ++i) {
                const float send = up ? q[i] : q[i + n / 2];
                const float keep = up ? q[i + n / 2] : q[i];
                q[i] = keep + __shfl_xor_sync(gmask, send, o);
              }
              n /= 2;
            } else {
              q[0] += __shfl_xor_sync(gmask, q[0], o);
            }
          }
          const int er_ = k0 + bu;
          const float sa = s_a[w][er_][bhead];
          const float dz = fabsf(sa) * (q[0] - s_d[w][er_][bhead]) * (signbit(sa) ? a.slope : 1.f);
          dacc += dz;
          if (bwriter) s_z[w][er_][bhead] = dz;
        } else {
          head_reduce<G, U, V, LPH>(p, gmask);
#pragma unroll
          for (int u = 0; u < U; ++u) {
            const int er_ = k0 + u;
#pragma unroll
            for (int v = 0; v < V; ++v) {
              const float sa = s_a[w][er_][hv[v]];
              const float dz = fabsf(sa) * (p[u][v] - s_d[w][er_][hv[v]]) * (signbit(sa) ? a.slope : 1.f);
              derv[v] += dz;
              if (head_lead<G, LPH>(gl, v)) s_z[w][er_][hv[v]] = dz;
            }
          }
        }
      }
      cp_async_wait<0>();  // the ring is empty between chunks (issue() past the chunk commits empty groups)
      __syncwarp();
      if (valid) {
        float *dzp = a.dz + (int64_t)cp_c * H;  // CSR order
        if constexpr (HT == 4) {
          st16f_pol(dzp, make_float4(s_z[w][lane][0], s_z[w][lane][1], s_z[w][lane][2], s_z[w][lane][3]), pol_st);
        } else {
          for (int h = 0; h < H; ++h) dzp[h] = s_z[w][lane][h];
        }
      }
      __syncwarp();
    }
    if constexpr (BFLY) {
      float dsum = dacc;
#pragma unroll
      for (int s = 0, o = LPH >> 1; s < UB; ++s, o >>= 1) dsum += __shfl_xor_sync(gmask, dsum, o);
#pragma unroll
      for (int v = 0; v < V; ++v) {
        int src = gl;
#pragma unroll
        for (int t = 0, o = LPH >> (1 + UB); (1 << t) < V; ++t, o >>= 1) {
          const int bit = (v >> ((V == 2 ? 1 : (V == 4 ? 2 : 3)) - 1 - t)) & 1;
          src = bit ? (src | o) : (src & ~o);
        }
        derv[v] = __shfl_sync(gmask, dsum, src);
      }
    }
    if (item.w < 0) {
      float *orow = a.gfeat + j * a.ldgf + gl * EPV;
#pragma unroll
      for (int v = 0; v < V; ++v) {
        const float *arp = a.ar + (v * G + gl) * EPV;
        float y[EPV];
#pragma unroll
        for (int k = 0; k < EPV; k += 4) {
          const float4 r4 = __ldg(reinterpret_cast<const float4 *>(arp + k));
          y[k] = fmaf(derv[v], r4.x, acc[v][k]); y[k + 1] = fmaf(derv[v], r4.y, acc[v][k + 1]);
          y[k + 2] = fmaf(derv[v], r4.z, acc[v][k + 2]); y[k + 3] = fmaf(derv[v], r4.w, acc[v][k + 3]);
          if (!a.lp_partial) st16f_pol(orow + v * G * EPV + k, make_float4(y[k], y[k + 1], y[k + 2], y[k + 3]), pol_st);
        }
        if (a.lp_partial) st16_pol(static_cast<T *>(a.gfeat_lp) + j * a.ldlp + (v * G + gl) * EPV, pack(y, T()), pol_st);
        if (head_lead<G, LPH>(gl, v)) a.der[j * H + hv[v]] = derv[v];
      }
    } else {
      const int64_t slot = item.w;
      float *pr = a.ws_bacc + slot * a.D + gl * EPV;
#pragma unroll
      for (int v = 0; v < V; ++v) {
#pragma unroll
        for (int k = 0; k < EPV; k += 4)
          *reinterpret_cast<float4 *>(pr + v * G * EPV + k) =
              make_float4(acc[v][k], acc[v][k + 1], acc[v][k + 2], acc[v][k + 3]);
        if (head_lead<G, LPH>(gl, v)) a.ws_bder[slot * H + hv[v]] = derv[v];
      }
    }
  }
}

// Split sources: dWh_j = sum_k acc_k + der_j a_r, der_j = sum_k der_k.
template <typename T, int G, int V>
__global__ void __launch_bounds__(TPB) gat_bwd_src_merge_kernel(const BwdArgs a) {
  constexpr int EPV = Tr<T>::EPV, GPW = 32 / G;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, gl = lane % G, grp = lane / G;
  const int H = a.H;
  const int64_t stride = (int64_t)gridDim.x * WPB * GPW;
  for (int64_t it = ((int64_t)blockIdx.x * WPB + w) * GPW + grp; it < a.L.n_bwd_splits; it += stride) {
    const int64_t j = a.L.bwd_splits[3 * it];
    const int s0 = a.L.bwd_splits[3 * it + 1], ns = a.L.bwd_splits[3 * it + 2];
    for (int h = gl; h < H; h += G) {
      float der = 0.f;
      for (int s = 0; s < ns; ++s) der += a.ws_bder[(int64_t)(s0 + s) * H + h];
      a.der[j * H + h] = der;
    }
#pragma unroll
    for (int v = 0; v < V; ++v) {
      const int col = (v * G + gl) * EPV, h = col / a.F;
      float der = 0.f, y[EPV];
#pragma unroll
      for (int k = 0; k < EPV; ++k) y[k] = 0.f;
      for (int s = 0; s < ns; ++s) {
        der += a.ws_bder[(int64_t)(s0 + s) * H + h];
        const float *pa = a.ws_bacc + (int64_t)(s0 + s) * a.D + col;
#pragma unroll
        for (int k = 0; k < EPV; ++k) y[k] += pa[k];
      }
      float *orow = a.gfeat + j * a.ldgf + col;
#pragma unroll
      for (int k = 0; k < EPV; ++k) y[k] = fmaf(der, a.ar[col + k], y[k]);
      if (a.lp_partial) {
        st16(static_cast<T *>(a.gfeat_lp) + j * a.ldlp + col, pack(y, T()));
      } else {
#pragma unroll
        for (int k = 0; k < EPV; ++k) orow[k] = y[k];
      }
    }
  }
}

// ---- a8: destination pass over this part's rows ----
// del_i = sum_In dz; dWh_i += del_i a_l; da_l += del_i Wh_i; da_r += der_i Wh_i.
template <typename T, int G, int V, int HT>
__global__ void __launch_bounds__(TPB, (V >= 4 ? 1 : (V == 2 ? 2 : 3))) gat_bwd_dst_kernel(const BwdArgs a) {
  constexpr int EPV = Tr<T>::EPV, FF = G * V * EPV / HT, LPH = FF / EPV, GPW = 32 / G;
  __shared__ double s_red[1024];
  __shared__ __align__(16) float s_dz[2][WPB][32][HT];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, gl = lane % G, grp = lane / G;
  const unsigned gmask = G == 32 ? 0xffffffffu : (((1u << G) - 1u) << (grp * G));
  constexpr int H = HT;   // heads is a power of two <= 8, dispatched as HT == heads (check_shape)
  const int rb = grp * G;
  int hv[V];
  float dal[V][EPV], dar[V][EPV], alv[V][EPV];
#pragma unroll
  for (int v = 0; v < V; ++v) {
    hv[v] = ((v * G + gl) * EPV) / FF;
#pragma unroll
    for (int k = 0; k < EPV; ++k) { dal[v][k] = 0.f; dar[v][k] = 0.f; alv[v][k] = a.al[(v * G + gl) * EPV + k]; }
  }
  const T *feat = static_cast<const T *>(a.feat);
  const int64_t stride = (int64_t)gridDim.x * WPB * GPW;
  // software pipeline over this group's rows: row k+1's first G dz values are
  // staged in shared memory with cp.async (each lane copies and reads back its
  // own slot: no barriers) and row k+2's indptr pair is loaded, while row k runs
  auto stage_dz = [&](int b, int e0, int e1) {
    if (e0 + gl < e1) cp_async_h<HT>(&s_dz[b][w][rb + gl][0], a.dz + (int64_t)(e0 + gl) * H);
    cp_async_commit();
  };
  // rows are taken in the layout's balanced order (dorder: descending in-degree, so each stride
  // round holds rows of similar work and no warp is left with the long ones at the end); this pass
  // gathers nothing, so the order costs no locality
  const int32_t *ord = a.L.dorder;
  auto row_at = [&](int64_t q) -> int64_t { return ord ? (int64_t)ord[q] : q; };
  int64_t pos = ((int64_t)blockIdx.x * WPB + w) * GPW + grp;
  // row ids and their indptr pairs are software-pipelined one and two rows ahead (cr, nr)
  int ce0 = 0, ce1 = 0, ne0 = 0, ne1 = 0, buf = 0;
  int64_t cr = 0, nr = 0;
  if (pos < a.L.rows) { cr = row_at(pos); ce0 = a.L.indptr[cr]; ce1 = a.L.indptr[cr + 1]; }
  stage_dz(0, ce0, ce1);
  if (pos + stride < a.L.rows) { nr = row_at(pos + stride); ne0 = a.L.indptr[nr]; ne1 = a.L.indptr[nr + 1]; }
  for (; pos < a.L.rows; pos += stride) {
    const int64_t r = cr;
    const int64_t grow = a.L.row_begin + r;
    // row-local operands first: they do not depend on del, so their latency
    // overlaps the dz gather below
    float *gr = a.gfeat + grow * a.ldgf + gl * EPV;
    const T *wr = feat + grow * a.ldf + gl * EPV;
    float4 part[V][EPV / 4];
    uint4 whp[V], plp[V];
#pragma unroll
    for (int v = 0; v < V; ++v) {
      whp[v] = ldg16(wr + v * G * EPV);
      if (a.lp_partial) {   // the source pass left its partial in the bf16 operand (read back, in place)
        plp[v] = *reinterpret_cast<const uint4 *>(static_cast<const T *>(a.gfeat_lp) + grow * a.ldlp + (v * G + gl) * EPV);
      } else {
#pragma unroll
        for (int k = 0; k < EPV / 4; ++k) part[v][k] = *reinterpret_cast<const float4 *>(gr + v * G * EPV + 4 * k);
      }
    }
    float derr[HT];
    load_h<HT>(a.der + grow * H, H, derr);
    const int e0 = ce0, e1 = ce1;
    if (pos + stride < a.L.rows) stage_dz(buf ^ 1, ne0, ne1);
    else cp_async_commit();
    ce0 = ne0; ce1 = ne1; cr = nr;
    if (pos + 2 * stride < a.L.rows) {
      nr = row_at(pos + 2 * stride);
      ne0 = a.L.indptr[nr];
      ne1 = a.L.indptr[nr + 1];
    }
    cp_async_wait<1>();  // this row's staged dz
    float dp[HT];
#pragma unroll
    for (int h = 0; h < HT; ++h) dp[h] = e0 + gl < e1 ? s_dz[buf][w][rb + gl][h] : 0.f;
    buf ^= 1;
    for (int e = e0 + G + gl; e < e1; e += G) {
      float t[HT];
      load_h<HT>(a.dz + (int64_t)e * H, H, t);  // dz is stored in CSR order by the source pass
#pragma unroll
      for (int h = 0; h < HT; ++h)
        if (h < H) dp[h] += t[h];
    }
    float del[HT];
#pragma unroll
    for (int h = 0; h < HT; ++h) del[h] = h < H ? gsum<G>(dp[h], gmask) : 0.f;
#pragma unroll
    for (int v = 0; v < V; ++v) {
      const float d = sel<HT>(del, hv[v]), dr = sel<HT>(derr, hv[v]);
      float y[EPV], wh[EPV];
      unpack(whp[v], wh, T());
      if (a.lp_partial) {   // unpacked only now: its load latency overlapped the dz gather
        float x[EPV];
        unpack(plp[v], x, T());
#pragma unroll
        for (int k = 0; k < EPV / 4; ++k) part[v][k] = make_float4(x[4 * k], x[4 * k + 1], x[4 * k + 2], x[4 * k + 3]);
      }
#pragma unroll
      for (int k = 0; k < EPV / 4; ++k) {
        y[4 * k] = fmaf(d, alv[v][4 * k], part[v][k].x);
        y[4 * k + 1] = fmaf(d, alv[v][4 * k + 1], part[v][k].y);
        y[4 * k + 2] = fmaf(d, alv[v][4 * k + 2], part[v][k].z);
        y[4 * k + 3] = fmaf(d, alv[v][4 * k + 3], part[v][k].w);
        if (!a.lp_only)
          *reinterpret_cast<float4 *>(gr + v * G * EPV + 4 * k) =
              make_float4(y[4 * k], y[4 * k + 1], y[4 * k + 2], y[4 * k + 3]);
      }
      if (a.gfeat_lp) st16(static_cast<T *>(a.gfeat_lp) + grow * a.ldlp + (v * G + gl) * EPV, pack(y, T()));
#pragma unroll
      for (int k = 0; k < EPV; ++k) {
        dal[v][k] = fmaf(d, wh[k], dal[v][k]);
        dar[v][k] = fmaf(dr, wh[k], dar[v][k]);
      }
    }
  }
  cp_async_wait<0>();
  block_partial<G, V, EPV>(dal, s_red, a.ws_dal + (int64_t)blockIdx.x * a.D, a.D);
  block_partial<G, V, EPV>(dar, s_red, a.ws_dar + (int64_t)blockIdx.x * a.D, a.D);
}

// Second stage of the parameter-gradient reductions (fixed order, fp64).
// Second stage of da_l (blockIdx.y = 0) and da_r (= 1): 32 columns per block, the
// per-CTA partials striped over 32 warps (fixed order: deterministic), then a
// shared-memory sum over the stripes.  One launch; the dependent-add chain per
// thread is nparts/32 long instead of nparts (the serial version cost ~19 us per
// call at nparts ~ 1.2K, most of a small-graph step).
__global__ void __launch_bounds__(1024) param_reduce_kernel(const double *parts_l, const double *parts_r,
                                                            int nparts, int D, float *out_l, float *out_r) {
  __shared__ double sh[32][33];
  const double *parts = blockIdx.y ? parts_r : parts_l;
  float *out = blockIdx.y ? out_r : out_l;
  const int tx = threadIdx.x & 31, ty = threadIdx.x >> 5;
  const int d = blockIdx.x * 32 + tx;
  double s = 0.0;
  if (d < D) {
#pragma unroll 4
    for (int b = ty; b < nparts; b += 32) s += parts[(int64_t)b * D + d];
  }
  sh[ty][tx] = s;
  __syncthreads();
  if (ty == 0 && d < D) {
    double t = 0.0;
#pragma unroll
    for (int k = 0; k < 32; ++k) t += sh[k][tx];
    out[d] = (float)t;
  }
}

// k-GPU exchange (SURVEY §8(e), NEXT-1 halo): dst[di] = src[si] for i < cnt, rows of
// row_bytes, si = sidx ? sidx[i] : i (gather into a send buffer), di = didx ? didx[i] : i
// (scatter out of a receive buffer).  16-byte vectors when everything is 16-byte aligned.
__global__ void __launch_bounds__(256) rows_move_kernel(const char *src, int64_t src_ld, const int32_t *sidx,
                                                        char *dst, int64_t dst_ld, const int32_t *didx, int64_t cnt,
                                                        int row_bytes, int vec16) {
  const int per = vec16 ? row_bytes / 16 : row_bytes / 4;
  const int64_t total = cnt * per;
  for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < total; t += (int64_t)gridDim.x * blockDim.x) {
    const int64_t i = t / per;
    const int c = (int)(t % per);
    const int64_t si = sidx ? sidx[i] : i, di = didx ? didx[i] : i;
    if (vec16)
      reinterpret_cast<uint4 *>(dst + di * dst_ld)[c] = reinterpret_cast<const uint4 *>(src + si * src_ld)[c];
    else
      reinterpret_cast<uint32_t *>(dst + di * dst_ld)[c] = reinterpret_cast<const uint32_t *>(src + si * src_ld)[c];
  }
}

// k-GPU backward: add the peers' partial [dWh | der] of this part's own rows (received rows
// `recv` [n][D] / `recv_der` [n][H]; pos[slot][r] = index of peer slot's partial of own row r,
// -1 if that peer has no edge from r) to the local partial, peers in ascending order (fixed
// order: deterministic).
__global__ void __launch_bounds__(256) dist_combine_kernel(float *gfeat, int64_t ldgf, float *der, const float *recv,
                                                           const float *recv_der, const int32_t *pos, int npeers,
                                                           int64_t rows, int64_t row0, int D, int H) {
  const int64_t nv = rows * (D / 4);
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nv; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = i / (D / 4), c = 4 * (i % (D / 4));
    float4 *dst = reinterpret_cast<float4 *>(gfeat + (row0 + r) * ldgf + c);
    float4 acc = *dst;
    for (int q = 0; q < npeers; ++q) {
      const int32_t t = pos[(int64_t)q * rows + r];
      if (t < 0) continue;
      const float4 v = *reinterpret_cast<const float4 *>(recv + (int64_t)t * D + c);
      acc.x += v.x; acc.y += v.y; acc.z += v.z; acc.w += v.w;
    }
    *dst = acc;
  }
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < rows * H; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = i / H, h = i % H;
    float acc = der[row0 * H + i];
    for (int q = 0; q < npeers; ++q) {
      const int32_t t = pos[(int64_t)q * rows + r];
      if (t >= 0) acc += recv_der[(int64_t)t * H + h];
    }
    der[row0 * H + i] = acc;
  }
}

}  // namespace kern

// ============================ host side ============================
namespace {
using namespace kern;

template <int X> using IC = std::integral_constant<int, X>;

// (G, V) for a row of `nv` 16-byte vectors.
template <typename Fn>
bool dispatch_gv(int nv, Fn &&fn) {
  switch (nv) {
    case 1: fn(IC<1>(), IC<1>()); return true;
    case 2: fn(IC<2>(), IC<1>()); return true;
    case 4: fn(IC<4>(), IC<1>()); return true;
    case 8: fn(IC<8>(), IC<1>()); return true;
    case 16: fn(IC<16>(), IC<1>()); return true;
    case 32: fn(IC<32>(), IC<1>()); return true;
    case 64: fn(IC<32>(), IC<2>()); return true;
    case 128: fn(IC<32>(), IC<4>()); return true;
    case 256: fn(IC<32>(), IC<8>()); return true;
    default: return false;
  }
}
// HT = heads rounded up to a power of two (<= 8)
template <typename Fn>
void dispatch_h(int H, Fn &&fn) {
  if (H <= 1) fn(IC<1>());
  else if (H <= 2) fn(IC<2>());
  else if (H <= 4) fn(IC<4>());
  else fn(IC<8>());
}

struct DevInfo { int sms = 0; int major = 0; };
DevInfo dev_info(int dev) {
  static std::mutex mu;
  static std::unordered_map<int, DevInfo> cache;
  std::lock_guard<std::mutex> g(mu);
  auto it = cache.find(dev);
  if (it != cache.end()) return it->second;
  DevInfo d;
  cudaDeviceGetAttribute(&d.sms, cudaDevAttrMultiProcessorCount, dev);
  cudaDeviceGetAttribute(&d.major, cudaDevAttrComputeCapabilityMajor, dev);
  cache[dev] = d;
  return d;
}

template <typename K>
int grid_for(K kernel, int64_t groups, int gpw, int dev) {
  static std::mutex mu;
  static std::unordered_map<const void *, int> occ;
  int per_sm;
  {
    std::lock_guard<std::mutex> g(mu);
    auto it = occ.find((const void *)kernel);
    if (it == occ.end()) {
      int nb = 0;
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, kernel, TPB, 0);
      per_sm = nb > 0 ? nb : 1;
      occ[(const void *)kernel] = per_sm;
    } else {
      per_sm = it->second;
    }
  }
  const int64_t need = (groups + (int64_t)WPB * gpw - 1) / ((int64_t)WPB * gpw);
  int64_t g = std::min<int64_t>(need, (int64_t)per_sm * dev_info(dev).sms);
  g = std::min<int64_t>(g, MAX_GRID);
  return (int)std::max<int64_t>(g, 1);
}

bool debug_sync() {
  static int v = -1;
  if (v < 0) {
    const char *e = std::getenv("MEGA_DEBUG_SYNC");
    v = (e && e[0] == '1') ? 1 : 0;
  }
  return v == 1;
}

int st_hint_mode() {   // MEGA_ST_HINT=0 turns the evict_first hints on streamed results off (ablation)
  static int v = -1;
  if (v < 0) {
    const char *e = std::getenv("MEGA_ST_HINT");
    v = e ? std::atoi(e) : 1;
  }
  return v;
}
mega_status check_launch(cudaStream_t s, const char *what) {
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return fail(MEGA_ERR_CUDA, std::string(what) + ": " + cudaGetErrorString(e));
  cudaStreamCaptureStatus cap = cudaStreamCaptureStatusNone;
  if (debug_sync() && cudaStreamIsCapturing(s, &cap) == cudaSuccess && cap == cudaStreamCaptureStatusNone) {
    e = cudaStreamSynchronize(s);  // never inside a CUDA-graph capture (illegal there)
    if (e != cudaSuccess) return fail(MEGA_ERR_CUDA, std::string(what) + " (sync): " + cudaGetErrorString(e));
  }
  return MEGA_OK;
}

size_t align256(size_t x) { return (x + 255) / 256 * 256; }

struct Shape {
  int H, F, D, epv, nv, G, V;
};

mega_status check_shape(int heads, int head_dim, mega_dtype dtype, Shape &s) {
  if (dtype != MEGA_F32 && dtype != MEGA_BF16) return fail(MEGA_ERR_INVALID_ARGUMENT, "dtype must be MEGA_F32 or MEGA_BF16");
  if (heads < 1 || heads > MAXH || (heads & (heads - 1)))
    return fail(MEGA_ERR_UNSUPPORTED, "heads must be 1, 2, 4 or 8");
  if (head_dim < 1) return fail(MEGA_ERR_INVALID_ARGUMENT, "head_dim must be >= 1");
  s.H = heads; s.F = head_dim; s.D = heads * head_dim;
  s.epv = dtype == MEGA_BF16 ? 8 : 4;
  if (head_dim % s.epv) return fail(MEGA_ERR_UNSUPPORTED, "head_dim must be a multiple of 8 (bf16) / 4 (fp32)");
  if (s.D > 1024) return fail(MEGA_ERR_UNSUPPORTED, "heads*head_dim must be <= 1024");
  s.nv = s.D / s.epv;
  bool ok = dispatch_gv(s.nv, [&](auto g, auto v) { s.G = decltype(g)::value; s.V = decltype(v)::value; });
  if (!ok) return fail(MEGA_ERR_UNSUPPORTED, "D/EPV must be a power of two <= 32 or 64/128/256");
  const int lph = s.F / s.epv;
  if (lph <= s.G) {
    if ((lph & (lph - 1)) || s.G % lph) return fail(MEGA_ERR_UNSUPPORTED, "head_dim/EPV must be a power of two");
  } else if (lph % s.G || s.V % (lph / s.G)) {
    return fail(MEGA_ERR_UNSUPPORTED, "unsupported head_dim for this row width");
  }
  return MEGA_OK;
}

bool al16(const void *p) { return (reinterpret_cast<uintptr_t>(p) & 15) == 0; }

mega_status check_part(const mega_layout *L, int32_t part, int &dev) {
  if (!L) return fail(MEGA_ERR_INVALID_ARGUMENT, "null layout");
  if (part < 0 || part >= (int32_t)L->parts.size()) return fail(MEGA_ERR_INVALID_ARGUMENT, "part out of range");
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return fail(MEGA_ERR_CUDA, std::string("cudaGetDevice: ") + cudaGetErrorString(e));
  if (dev_info(dev).major != 10) return fail(MEGA_ERR_UNSUPPORTED, "libmega.so kernels require an sm_100 (B200) device");
  const Part &P = L->parts[part];
  if (!P.dev_base) return fail(MEGA_ERR_STATE, "layout part not bound (mega_layout_bind_device)");
  if (P.device != dev) return fail(MEGA_ERR_STATE, "layout part bound to another device");
  return MEGA_OK;
}

// work-claim counters (one per claiming launch of a call), zeroed at the start of the call
constexpr int kCtrs = 64;
struct WsFwd { size_t m, l, acc, ctr, total; };
WsFwd ws_fwd(const DevPart &D, const Shape &s) {
  WsFwd w;
  size_t slots = (size_t)std::max(1, D.n_fwd_slots);
  w.m = 0;
  w.l = align256(w.m + slots * s.H * 4);
  w.acc = align256(w.l + slots * s.H * 4);
  w.ctr = align256(w.acc + slots * s.D * 4);
  w.total = align256(w.ctr + kCtrs * 4);
  return w;
}
// MEGA_LP_PARTIAL=0: keep the source pass's dWh partial in fp32 grad_feat in LP_ONLY mode (ablation)
bool lp_partial_mode() {
  static int v = -1;
  if (v < 0) {
    const char *e = std::getenv("MEGA_LP_PARTIAL");
    v = e ? std::atoi(e) : 1;
  }
  return v != 0;
}
// Claiming pays once a launch has many rounds of chunks to hand out: with few (the paper's small
// batches, ~50 chunks) every group takes at most a chunk or two, the warps cannot drift apart, and the
// counter reset plus the claim -> bounds -> descriptor chain only add latency to a launch-bound step
// (zinc-b64: 0.17 -> 0.27 ms/step with claiming everywhere).
bool claim_pays(int64_t n_chunks, int dev) { return n_chunks >= 16 * 16 * (int64_t)dev_info(dev).sms; }
// MEGA_SCHED_DYN=0: static striding over the chunks instead of claiming them (ablation)
bool sched_dynamic() {
  static int v = -1;
  if (v < 0) {
    const char *e = std::getenv("MEGA_SCHED_DYN");
    v = e ? std::atoi(e) : 1;
  }
  return v != 0;
}
struct WsBwd { size_t dz, bacc, bder, dal, dar, ctr, total; };
WsBwd ws_bwd(const DevPart &D, const Shape &s) {
  WsBwd w;
  size_t slots = (size_t)std::max(1, D.n_bwd_slots);
  w.dz = 0;
  w.bacc = align256(w.dz + (size_t)std::max<int64_t>(1, D.edges) * s.H * 4);
  w.bder = align256(w.bacc + slots * s.D * 4);
  w.dal = align256(w.bder + slots * s.H * 4);
  w.dar = align256(w.dal + (size_t)MAX_GRID * s.D * 8);
  w.ctr = align256(w.dar + (size_t)MAX_GRID * s.D * 8);
  w.total = align256(w.ctr + kCtrs * 4);
  return w;
}
DevPart host_counts(const Part &P, int64_t n) {  // sizes without binding
  DevPart D;
  D.n = n;
  D.rows = P.row_end - P.row_begin;
  D.edges = (int64_t)P.src.size();
  D.n_fwd_slots = P.n_fwd_slots;
  D.n_bwd_slots = P.n_bwd_slots;
  return D;
}

template <typename T>
mega_status launch_eler(const void *feat, int64_t ldf, int64_t rows, int64_t row0, const float *al, const float *ar,
                        const Shape &s, float *el, float *er, cudaStream_t st, int dev) {
  mega_status rc = MEGA_OK;
  dispatch_gv(s.nv, [&](auto g, auto v) {
    constexpr int G = decltype(g)::value, V = decltype(v)::value;
    dispatch_h(s.H, [&](auto ht) {
      auto k = eler_kernel<T, G, V, decltype(ht)::value>;
      const int grid = grid_for(k, rows, 32 / G, dev);
      k<<<grid, TPB, 0, st>>>(static_cast<const T *>(feat), ldf, rows, row0, al, ar, s.H, s.F, el, er);
      rc = check_launch(st, "eler_kernel");
    });
  });
  return rc;
}

}  // namespace

// internal entry used by project.cu
mega_status launch_eler_any(mega_dtype dt, const void *feat, int64_t ldf, int64_t rows, int64_t row0, const float *al,
                            const float *ar, int heads, int head_dim, float *el, float *er, cudaStream_t st) {
  Shape s;
  mega_status rc = check_shape(heads, head_dim, dt, s);
  if (rc != MEGA_OK) return rc;
  int dev = 0;
  cudaGetDevice(&dev);
  if (rows == 0) return MEGA_OK;
  return dt == MEGA_BF16 ? launch_eler<__nv_bfloat16>(feat, ldf, rows, row0, al, ar, s, el, er, st, dev)
                         : launch_eler<float>(feat, ldf, rows, row0, al, ar, s, el, er, st, dev);
}

namespace {
template <typename T>
mega_status run_fwd(const FwdArgs &a, const Shape &s, cudaStream_t st, int dev) {
  mega_status rc = MEGA_OK;
  dispatch_gv(s.nv, [&](auto g, auto v) {
    constexpr int G = decltype(g)::value, V = decltype(v)::value;
    if (a.L.n_fwd_items > 0) {
      dispatch_h(s.H, [&](auto ht) {
        constexpr int HT = decltype(ht)::value;
        auto launch = [&](auto kern_fn) {
          kern_fn<<<grid_for(kern_fn, a.L.n_fwd_items, 32 / G, dev), TPB, 0, st>>>(a);
          rc = check_launch(st, "gat_fwd_kernel");
        };
        // chunk-pipelined kernel for groups of >= 8 lanes (products 3 layers: 25.5 vs 29.3 ms/step for the
        // register-batch kernel, which stays for narrow rows: static shared memory of the pipe kernel).
        // A TMA-ring variant (rows in flight in shared memory, cp.async.bulk per row) measured 9.7 vs
        // 6.8 ms per products layer: 113 vs 85 warp instructions per edge in an issue-bound kernel
        if constexpr (G >= 8) launch(gat_fwd_pipe_kernel<T, G, V, HT>);
        else launch(gat_fwd_kernel<T, G, V, HT, 0>);
      });
      if (rc != MEGA_OK) return;
    }
    if (a.L.n_fwd_splits > 0) {
      auto k = gat_fwd_merge_kernel<T, G, V>;
      k<<<grid_for(k, a.L.n_fwd_splits, 32 / G, dev), TPB, 0, st>>>(a);
      rc = check_launch(st, "gat_fwd_merge_kernel");
    }
  });
  return rc;
}

template <typename T>
mega_status run_bwd(BwdArgs a, const Shape &s, uint32_t flags, cudaStream_t st, int dev, bool with_dlt = true) {
  mega_status rc = MEGA_OK;
  const uint32_t ph = flags & (MEGA_BWD_PHASE_SRC | MEGA_BWD_PHASE_DST);
  const bool src_phase = ph == 0 || (ph & MEGA_BWD_PHASE_SRC);
  const bool dst_phase = ph == 0 || (ph & MEGA_BWD_PHASE_DST);
  dispatch_gv(s.nv, [&](auto g, auto v) {
    constexpr int G = decltype(g)::value, V = decltype(v)::value;
    dispatch_h(s.H, [&](auto ht) {
      constexpr int HT = decltype(ht)::value;
      if (src_phase) {
        if (with_dlt && a.L.rows > 0) {
          auto k = dlt_kernel<T, G, V, HT>;
          k<<<grid_for(k, a.L.rows, 32 / G, dev), TPB, 0, st>>>(a);
          if ((rc = check_launch(st, "dlt_kernel")) != MEGA_OK) return;
        }
        if (a.L.n_bwd_items > 0) {
          bool ring = false;
          if constexpr (G == 32 && V <= 2) {
            // shared-memory ring, NBF batches of U rows in flight: (U, NBF) = (4, 2) for 2 vectors per lane,
            // (8, 2) for 1 (round 1: (2, 4) / (4, 4)); products per step gat_bwd_src 34.2 -> 31.4 ms, reddit
            // 8.3 -> 7.6; (2 U, 3) and (U / 2, 6) measured slower (profiles/r02/ring/)
            constexpr int U = V == 2 ? 4 : 8, NBF = 2;
            auto kr = gat_bwd_src_ring_kernel<T, V, HT, U, NBF>;
            const size_t smem = (size_t)WPB * NBF * U * V * 32 * 16;
            cudaFuncSetAttribute(kr, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
            int nblk = 0;
            cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nblk, kr, TPB, smem);
            const int grid = (int)std::min<int64_t>((a.L.n_bwd_items + WPB - 1) / WPB,
                                                    (int64_t)dev_info(dev).sms * std::max(nblk, 1));
            kr<<<std::max(grid, 1), TPB, smem, st>>>(a);
            ring = true;
          }
          if (!ring) {
            auto ks = gat_bwd_src_kernel<T, G, V, HT, 0>;
            ks<<<grid_for(ks, a.L.n_bwd_items, 32 / G, dev), TPB, 0, st>>>(a);
          }
          if ((rc = check_launch(st, "gat_bwd_src_kernel")) != MEGA_OK) return;
        }
        if (a.L.n_bwd_splits > 0) {
          auto km = gat_bwd_src_merge_kernel<T, G, V>;
          km<<<grid_for(km, a.L.n_bwd_splits, 32 / G, dev), TPB, 0, st>>>(a);
          if ((rc = check_launch(st, "gat_bwd_src_merge_kernel")) != MEGA_OK) return;
        }
      }
      if (dst_phase) {
        auto kd = gat_bwd_dst_kernel<T, G, V, HT>;
        a.nb_dst = grid_for(kd, std::max<int64_t>(1, a.L.rows), 32 / G, dev);
        kd<<<a.nb_dst, TPB, 0, st>>>(a);
        if ((rc = check_launch(st, "gat_bwd_dst_kernel")) != MEGA_OK) return;
        param_reduce_kernel<<<dim3((s.D + 31) / 32, 2), 1024, 0, st>>>(a.ws_dal, a.ws_dar, a.nb_dst, s.D, a.gal,
                                                                       a.gar);
        rc = check_launch(st, "param_reduce_kernel");
      }
    });
  });
  return rc;
}
}  // namespace
}  // namespace mega

using namespace mega;

extern "C" {

mega_status mega_gat_workspace_bytes(const mega_layout *L, int32_t part, int heads, int head_dim, mega_dtype dtype,
                                     size_t *fwd_ws, size_t *bwd_ws) {
  clear_error();
  if (!L || !fwd_ws || !bwd_ws) return fail(MEGA_ERR_INVALID_ARGUMENT, "null argument");
  if (part < 0 || part >= (int32_t)L->parts.size()) return fail(MEGA_ERR_INVALID_ARGUMENT, "part out of range");
  Shape s;
  mega_status rc = check_shape(heads, head_dim, dtype, s);
  if (rc != MEGA_OK) return rc;
  DevPart D = host_counts(L->parts[part], L->n);
  *fwd_ws = ws_fwd(D, s).total;
  *bwd_ws = ws_bwd(D, s).total;
  return MEGA_OK;
}

mega_status mega_gat_fwd(const mega_layout *L, int32_t part, const void *feat, int64_t ldf, const float *attn_l,
                         const float *attn_r, int heads, int head_dim, mega_dtype dtype, float negative_slope,
                         uint32_t flags, void *out, int64_t ldo, float *ctx, void *ws, size_t ws_bytes,
                         mega_stream_t stream) {
  clear_error();
  NvtxRange nvtx_("mega_gat_fwd");
  int dev = 0;
  mega_status rc = check_part(L, part, dev);
  if (rc != MEGA_OK) return rc;
  Shape s;
  if ((rc = check_shape(heads, head_dim, dtype, s)) != MEGA_OK) return rc;
  if (!feat || !attn_l || !attn_r || !out || !ctx || !ws) return fail(MEGA_ERR_INVALID_ARGUMENT, "null pointer");
  const int esz = dtype == MEGA_BF16 ? 2 : 4;
  if (ldf < s.D || ldo < s.D || (ldf * esz) % 16 || (ldo * esz) % 16)
    return fail(MEGA_ERR_INVALID_ARGUMENT, "ldf/ldo must be >= D and a multiple of 16 bytes");
  if ((uint64_t)L->n * (uint64_t)ldf >= (1ULL << 32))
    return fail(MEGA_ERR_UNSUPPORTED, "num_nodes * ldf must be < 2^32 elements (32-bit row offsets)");
  if (!al16(feat) || !al16(out) || !al16(ctx) || !al16(ws)) return fail(MEGA_ERR_INVALID_ARGUMENT, "pointers must be 16-byte aligned");
  const Part &P = L->parts[part];
  const WsFwd w = ws_fwd(P.dev, s);
  if (ws_bytes < w.total) return fail(MEGA_ERR_OUT_OF_MEMORY, "fwd workspace too small");
  cudaStream_t st = (cudaStream_t)stream;
  const int64_t n = L->n, plane = n * s.H;
  if (!(flags & MEGA_FLAG_ELER_IN_CTX)) {
    rc = launch_eler_any(dtype, feat, ldf, n, 0, attn_l, attn_r, heads, head_dim, ctx, ctx + plane, st);
    if (rc != MEGA_OK) return rc;
  }
  kern::FwdArgs a;
  a.L = P.dev;
  a.feat = feat; a.ldf = ldf;
  a.el = ctx; a.er = ctx + plane; a.lse = ctx + 2 * plane;
  a.H = s.H; a.F = s.F; a.D = s.D; a.slope = negative_slope;
  a.out = out; a.ldo = ldo;
  char *wb = static_cast<char *>(ws);
  a.ws_m = reinterpret_cast<float *>(wb + w.m);
  a.ws_l = reinterpret_cast<float *>(wb + w.l);
  a.ws_acc = reinterpret_cast<float *>(wb + w.acc);
  a.st_hint = st_hint_mode();
  a.ctr = nullptr;
  if (sched_dynamic() && claim_pays(P.dev.fchunk ? P.dev.n_fchunks : P.dev.n_fwd_items, dev)) {
    a.ctr = reinterpret_cast<int *>(wb + w.ctr);
    cudaError_t ce = cudaMemsetAsync(a.ctr, 0, kCtrs * 4, st);
    if (ce != cudaSuccess) return fail(MEGA_ERR_CUDA, std::string("counter reset: ") + cudaGetErrorString(ce));
  }
  return dtype == MEGA_BF16 ? run_fwd<__nv_bfloat16>(a, s, st, dev) : run_fwd<float>(a, s, st, dev);
}

mega_status mega_gat_bwd(const mega_layout *L, int32_t part, const void *feat, int64_t ldf, const float *attn_l,
                         const float *attn_r, int heads, int head_dim, mega_dtype dtype, float negative_slope,
                         uint32_t flags, const void *out, int64_t ldo, const void *grad_out, int64_t ldg, float *ctx,
                         float *grad_feat, int64_t ldgf, void *grad_feat_lp, int64_t ldlp, float *grad_attn_l,
                         float *grad_attn_r, void *ws, size_t ws_bytes, mega_stream_t stream) {
  clear_error();
  NvtxRange nvtx_("mega_gat_bwd");
  int dev = 0;
  mega_status rc = check_part(L, part, dev);
  if (rc != MEGA_OK) return rc;
  Shape s;
  if ((rc = check_shape(heads, head_dim, dtype, s)) != MEGA_OK) return rc;
  if (!feat || !attn_l || !attn_r || !out || !grad_out || !ctx || !grad_feat || !grad_attn_l || !grad_attn_r || !ws)
    return fail(MEGA_ERR_INVALID_ARGUMENT, "null pointer");
  const int esz = dtype == MEGA_BF16 ? 2 : 4;
  if (ldf < s.D || ldo < s.D || ldg < s.D || ldgf < s.D || (ldf * esz) % 16 || (ldo * esz) % 16 || (ldg * esz) % 16 ||
      (ldgf * 4) % 16)
    return fail(MEGA_ERR_INVALID_ARGUMENT, "leading dimensions must be >= D and multiples of 16 bytes");
  if ((uint64_t)L->n * (uint64_t)std::max(ldf, ldg) >= (1ULL << 32))
    return fail(MEGA_ERR_UNSUPPORTED, "num_nodes * ld must be < 2^32 elements (32-bit row offsets)");
  if (grad_feat_lp && (ldlp < s.D || (ldlp * esz) % 16 || !al16(grad_feat_lp)))
    return fail(MEGA_ERR_INVALID_ARGUMENT, "grad_feat_lp: bad ld or alignment");
  if (!al16(feat) || !al16(out) || !al16(grad_out) || !al16(ctx) || !al16(grad_feat) || !al16(ws) ||
      !al16(attn_l) || !al16(attn_r))
    return fail(MEGA_ERR_INVALID_ARGUMENT, "pointers must be 16-byte aligned");
  const Part &P = L->parts[part];
  const WsBwd w = ws_bwd(P.dev, s);
  if (ws_bytes < w.total) return fail(MEGA_ERR_OUT_OF_MEMORY, "bwd workspace too small");
  const int64_t plane = L->n * s.H;
  kern::BwdArgs a;
  a.L = P.dev;
  a.feat = feat; a.ldf = ldf; a.al = attn_l; a.ar = attn_r;
  a.H = s.H; a.F = s.F; a.D = s.D; a.slope = negative_slope;
  a.out = out; a.ldo = ldo; a.gout = grad_out; a.ldg = ldg;
  a.el = ctx; a.er = ctx + plane; a.lse = ctx + 2 * plane; a.dlt = ctx + 3 * plane; a.der = ctx + 4 * plane;
  a.gfeat = grad_feat; a.ldgf = ldgf; a.gfeat_lp = grad_feat_lp; a.ldlp = ldlp;
  char *wb = static_cast<char *>(ws);
  a.dz = reinterpret_cast<float *>(wb + w.dz);
  a.ws_bacc = reinterpret_cast<float *>(wb + w.bacc);
  a.ws_bder = reinterpret_cast<float *>(wb + w.bder);
  a.ws_dal = reinterpret_cast<double *>(wb + w.dal);
  a.ws_dar = reinterpret_cast<double *>(wb + w.dar);
  a.gal = grad_attn_l; a.gar = grad_attn_r;
  a.nb_dst = 0;
  a.lp_only = (flags & MEGA_BWD_LP_ONLY) && grad_feat_lp ? 1 : 0;
  // LP_ONLY in bf16 with both phases in this call: the source pass leaves dWh's partial in the bf16
  // operand itself instead of fp32 grad_feat (DESIGN R-lp: 2.5 GB less written and read per products layer)
  a.lp_partial = a.lp_only && dtype == MEGA_BF16 && !(flags & (MEGA_BWD_PHASE_SRC | MEGA_BWD_PHASE_DST)) &&
                 lp_partial_mode() ? 1 : 0;
  a.st_hint = st_hint_mode();
  cudaStream_t st = (cudaStream_t)stream;
  a.ctr = nullptr;
  const uint32_t ph = flags & (MEGA_BWD_PHASE_SRC | MEGA_BWD_PHASE_DST);
  if (sched_dynamic() && (ph == 0 || (ph & MEGA_BWD_PHASE_SRC)) &&
      claim_pays(P.dev.bchunk ? P.dev.n_bchunks : P.dev.n_bwd_items, dev)) {
    a.ctr = reinterpret_cast<int *>(wb + w.ctr);
    cudaError_t ce = cudaMemsetAsync(a.ctr, 0, kCtrs * 4, st);
    if (ce != cudaSuccess) return fail(MEGA_ERR_CUDA, std::string("counter reset: ") + cudaGetErrorString(ce));
  }
  return dtype == MEGA_BF16 ? run_bwd<__nv_bfloat16>(a, s, flags, st, dev) : run_bwd<float>(a, s, flags, st, dev);
}

}  // extern "C"

// ---------------- k-GPU path ----------------
namespace mega {
namespace {
// workspace of the dist calls: fwd = mega_gat_fwd's (with the split-row slots) + halo send / receive
// buffers of packed [Wh | er] rows; bwd = mega_gat_bwd's + packed partial [dWh | der] rows out / in
struct DistWs { size_t fwd_base, f_sf, f_se, f_rf, f_re, fwd_total, bwd_base, b_sf, b_se, b_rf, b_re, bwd_total; };
DistWs dist_ws(const mega_layout *L, int32_t part, const Shape &s) {
  const Part &P = L->parts[part];
  DevPart D = host_counts(P, L->n);
  int32_t nslots = P.n_d_slots;
  int64_t nsend = (int64_t)P.hsend_idx.size(), nrecv = (int64_t)P.hrecv_idx.size();
  if (L->parts.size() > 1 && P.dl_items.empty() && P.dr_items.empty()) {
    std::vector<int32_t> a, b, c, d, e, f, g, h;
    dist_items(L, part, a, b, c, nslots);
    halo_plan(L, part, d, e, f, g, h);
    nsend = (int64_t)d.size();
    nrecv = (int64_t)f.size();
  }
  D.n_fwd_slots = std::max(D.n_fwd_slots, nslots);
  const size_t esz = 16 / s.epv, rf = (size_t)s.D * esz, re = (size_t)s.H * 4;
  DistWs w;
  w.fwd_base = ws_fwd(D, s).total;
  w.f_sf = w.fwd_base;
  w.f_se = align256(w.f_sf + nsend * rf);
  w.f_rf = align256(w.f_se + nsend * re);
  w.f_re = align256(w.f_rf + nrecv * rf);
  w.fwd_total = align256(w.f_re + nrecv * re);
  w.bwd_base = ws_bwd(D, s).total;
  w.b_sf = w.bwd_base;                                   // partials of the peers' rows this part references
  w.b_se = align256(w.b_sf + nrecv * (size_t)s.D * 4);
  w.b_rf = align256(w.b_se + nrecv * re);                // the peers' partials of this part's rows
  w.b_re = align256(w.b_rf + nsend * (size_t)s.D * 4);
  w.bwd_total = align256(w.b_re + nsend * re);
  return w;
}
mega_status move_rows(const void *src, int64_t src_ld, const int32_t *sidx, void *dst, int64_t dst_ld,
                      const int32_t *didx, int64_t cnt, int row_bytes, cudaStream_t st, int dev) {
  if (cnt <= 0) return MEGA_OK;
  const bool v16 = row_bytes % 16 == 0 && src_ld % 16 == 0 && dst_ld % 16 == 0 && al16(src) && al16(dst);
  const int64_t total = cnt * (v16 ? row_bytes / 16 : row_bytes / 4);
  const int blocks = (int)std::min<int64_t>((total + 255) / 256, 8 * dev_info(dev).sms);
  kern::rows_move_kernel<<<std::max(blocks, 1), 256, 0, st>>>(static_cast<const char *>(src), src_ld, sidx,
                                                               static_cast<char *>(dst), dst_ld, didx, cnt, row_bytes,
                                                               v16 ? 1 : 0);
  return check_launch(st, "rows_move_kernel");
}
bool phase_flags(uint32_t flags, bool &snd, bool &rcv) {
  const uint32_t ph = flags & (MEGA_DIST_PHASE_SEND | MEGA_DIST_PHASE_RECV);
  snd = ph == 0 || (ph & MEGA_DIST_PHASE_SEND);
  rcv = ph == 0 || (ph & MEGA_DIST_PHASE_RECV);
  return true;
}
mega_status check_comm(const mega_layout *L, int32_t part, mega_comm *c) {
  if (!c) return fail(MEGA_ERR_INVALID_ARGUMENT, "null comm");
  if (comm_size(c) != (int)L->parts.size())
    return fail(MEGA_ERR_INVALID_ARGUMENT, "comm size != layout num_parts");
  if (comm_rank(c) != part) return fail(MEGA_ERR_INVALID_ARGUMENT, "part must equal the comm rank");
  return MEGA_OK;
}
}  // namespace
}  // namespace mega

extern "C" {

mega_status mega_gat_dist_workspace_bytes(const mega_layout *L, int32_t part, int heads, int head_dim, mega_dtype dtype,
                                          size_t *fwd_ws, size_t *bwd_ws) {
  clear_error();
  if (!L || !fwd_ws || !bwd_ws) return fail(MEGA_ERR_INVALID_ARGUMENT, "null argument");
  if (part < 0 || part >= (int32_t)L->parts.size()) return fail(MEGA_ERR_INVALID_ARGUMENT, "part out of range");
  Shape s;
  mega_status rc = check_shape(heads, head_dim, dtype, s);
  if (rc != MEGA_OK) return rc;
  const DistWs w = dist_ws(L, part, s);
  *fwd_ws = w.fwd_total;
  *bwd_ws = w.bwd_total;
  return MEGA_OK;
}

mega_status mega_gat_fwd_dist(const mega_layout *L, int32_t part, mega_comm *comm, void *feat, int64_t ldf,
                              const float *attn_l, const float *attn_r, int heads, int head_dim, mega_dtype dtype,
                              float negative_slope, uint32_t flags, void *out, int64_t ldo, float *ctx, void *ws,
                              size_t ws_bytes, mega_stream_t stream, mega_stream_t comm_stream) {
  clear_error();
  NvtxRange nvtx_("mega_gat_fwd_dist");
  int dev = 0;
  mega_status rc = check_part(L, part, dev);
  if (rc != MEGA_OK) return rc;
  if ((rc = check_comm(L, part, comm)) != MEGA_OK) return rc;
  if (L->parts.size() == 1)   // nothing to exchange
    return mega_gat_fwd(L, part, feat, ldf, attn_l, attn_r, heads, head_dim, dtype, negative_slope,
                        flags & MEGA_FLAG_ELER_IN_CTX, out, ldo, ctx, ws, ws_bytes, stream);
  Shape s;
  if ((rc = check_shape(heads, head_dim, dtype, s)) != MEGA_OK) return rc;
  if (!feat || !attn_l || !attn_r || !out || !ctx || !ws) return fail(MEGA_ERR_INVALID_ARGUMENT, "null pointer");
  const int esz = dtype == MEGA_BF16 ? 2 : 4;
  if (ldf < s.D || ldo < s.D || (ldf * esz) % 16 || (ldo * esz) % 16)
    return fail(MEGA_ERR_INVALID_ARGUMENT, "ldf/ldo must be >= D and a multiple of 16 bytes");
  if ((uint64_t)L->n * (uint64_t)ldf >= (1ULL << 32))
    return fail(MEGA_ERR_UNSUPPORTED, "num_nodes * ldf must be < 2^32 elements (32-bit row offsets)");
  if (!al16(feat) || !al16(out) || !al16(ctx) || !al16(ws)) return fail(MEGA_ERR_INVALID_ARGUMENT, "pointers must be 16-byte aligned");
  const Part &P = L->parts[part];
  const DistWs dw = dist_ws(L, part, s);
  if (ws_bytes < dw.fwd_total) return fail(MEGA_ERR_OUT_OF_MEMORY, "fwd workspace too small (mega_gat_dist_workspace_bytes)");
  bool snd, rcv;
  phase_flags(flags, snd, rcv);
  cudaStream_t st = (cudaStream_t)stream, cs = (cudaStream_t)comm_stream;
  const int64_t n = L->n, plane = n * s.H, b0 = P.row_begin, rows = P.row_end - P.row_begin;
  char *fb = static_cast<char *>(feat);
  kern::FwdArgs a;
  a.L = P.dev;
  a.feat = feat; a.ldf = ldf;
  a.el = ctx; a.er = ctx + plane; a.lse = ctx + 2 * plane;
  a.H = s.H; a.F = s.F; a.D = s.D; a.slope = negative_slope;
  a.out = out; a.ldo = ldo;
  DevPart Dw = P.dev;
  Dw.n_fwd_slots = std::max(P.dev.n_fwd_slots, P.dev.n_d_slots);
  const WsFwd w = ws_fwd(Dw, s);
  char *wb = static_cast<char *>(ws);
  a.ws_m = reinterpret_cast<float *>(wb + w.m);
  a.ws_l = reinterpret_cast<float *>(wb + w.l);
  a.ws_acc = reinterpret_cast<float *>(wb + w.acc);
  a.st_hint = st_hint_mode();
  // counters: 0 = the local pass, 1 = the remote pass; zeroed by the SEND phase (the RECV phase may be
  // a separate call)
  int *ctrs = sched_dynamic() ? reinterpret_cast<int *>(wb + w.ctr) : nullptr;
  auto pass = [&](const int4 *items, int32_t nitems, const int32_t *splits, int32_t nsplits, int ci) {
    kern::FwdArgs b = a;
    b.ctr = ctrs ? ctrs + ci : nullptr;
    b.L.fwd_items = items; b.L.n_fwd_items = nitems; b.L.fchunk = nullptr;
    b.L.fwd_splits = splits; b.L.n_fwd_splits = nsplits;
    return dtype == MEGA_BF16 ? run_fwd<__nv_bfloat16>(b, s, st, dev) : run_fwd<float>(b, s, st, dev);
  };
  // NEXT-1 halo exchange: only the rows a peer's edges reference, packed [Wh] and [er] per peer
  const int k = (int)L->parts.size();
  const size_t rf = (size_t)s.D * esz, re = (size_t)s.H * 4;
  char *sf = wb + dw.f_sf, *se = wb + dw.f_se, *rfb = wb + dw.f_rf, *reb = wb + dw.f_re;
  std::vector<CommMsg> sends, recvs;
  for (int q = 0; q < k; ++q) {
    if (q == part) continue;
    const int64_t s0 = P.hsend_off[q], sn = P.hsend_off[q + 1] - s0, r0 = P.hrecv_off[q], rn = P.hrecv_off[q + 1] - r0;
    sends.push_back({q, 0, sf + s0 * rf, (size_t)sn * rf});
    sends.push_back({q, 1, se + s0 * re, (size_t)sn * re});
    recvs.push_back({q, 0, rfb + r0 * rf, (size_t)rn * rf});
    recvs.push_back({q, 1, reb + r0 * re, (size_t)rn * re});
  }
  const DevPart &DP = P.dev;
  if (snd) {
    if (!(flags & MEGA_FLAG_ELER_IN_CTX) && rows > 0) {   // el/er of the own rows (those we send)
      rc = launch_eler_any(dtype, fb + b0 * ldf * esz, ldf, rows, b0, attn_l, attn_r, heads, head_dim, ctx, ctx + plane, st);
      if (rc != MEGA_OK) return rc;
    }
    if (ctrs) {
      cudaError_t ce = cudaMemsetAsync(ctrs, 0, kCtrs * 4, st);
      if (ce != cudaSuccess) return fail(MEGA_ERR_CUDA, std::string("counter reset: ") + cudaGetErrorString(ce));
    }
    // pack the own rows the peers need, send them on the comm stream, receive the peers' rows ...
    if ((rc = move_rows(fb, ldf * esz, DP.hsend_idx, sf, rf, nullptr, DP.n_hsend, (int)rf, st, dev)) != MEGA_OK) return rc;
    if ((rc = move_rows(ctx + plane, re, DP.hsend_idx, se, re, nullptr, DP.n_hsend, (int)re, st, dev)) != MEGA_OK) return rc;
    if ((rc = comm_exchange(comm, sends, recvs, st, cs, true, false)) != MEGA_OK) return rc;
    // ... while block (p, p) (sources this rank owns) runs on the compute stream
    if ((rc = pass(DP.dl_items, DP.n_dl_items, nullptr, 0, 0)) != MEGA_OK) return rc;
  }
  if (rcv) {
    if ((rc = comm_exchange(comm, sends, recvs, st, cs, false, true)) != MEGA_OK) return rc;
    // scatter the received rows into the global [Wh | er] arrays (comm stream), then continue
    if ((rc = move_rows(rfb, rf, nullptr, fb, ldf * esz, DP.hrecv_idx, DP.n_hrecv, (int)rf, cs, dev)) != MEGA_OK) return rc;
    if ((rc = move_rows(reb, re, nullptr, ctx + plane, re, DP.hrecv_idx, DP.n_hrecv, (int)re, cs, dev)) != MEGA_OK) return rc;
    cudaError_t ce = cudaEventRecord(comm_done_event(comm), cs);
    if (ce == cudaSuccess) ce = cudaStreamWaitEvent(st, comm_done_event(comm), 0);
    if (ce != cudaSuccess) return fail(MEGA_ERR_CUDA, std::string("wait comm: ") + cudaGetErrorString(ce));
    // remote blocks, then the fixed-order merge of the rows split across passes / segments (KB7)
    if ((rc = pass(DP.dr_items, DP.n_dr_items, nullptr, 0, 1)) != MEGA_OK) return rc;
    if ((rc = pass(nullptr, 0, DP.d_splits, DP.n_d_splits, 2)) != MEGA_OK) return rc;
  }
  return MEGA_OK;
}

mega_status mega_gat_bwd_dist(const mega_layout *L, int32_t part, mega_comm *comm, const void *feat, int64_t ldf,
                              const float *attn_l, const float *attn_r, int heads, int head_dim, mega_dtype dtype,
                              float negative_slope, uint32_t flags, const void *out, int64_t ldo, const void *grad_out,
                              int64_t ldg, float *ctx, float *grad_feat, int64_t ldgf, void *grad_feat_lp,
                              int64_t ldlp, float *grad_attn_l, float *grad_attn_r, void *ws, size_t ws_bytes,
                              mega_stream_t stream, mega_stream_t comm_stream) {
  clear_error();
  NvtxRange nvtx_("mega_gat_bwd_dist");
  int dev = 0;
  mega_status rc = check_part(L, part, dev);
  if (rc != MEGA_OK) return rc;
  if ((rc = check_comm(L, part, comm)) != MEGA_OK) return rc;
  if (L->parts.size() == 1)
    return mega_gat_bwd(L, part, feat, ldf, attn_l, attn_r, heads, head_dim, dtype, negative_slope,
                        flags & MEGA_BWD_LP_ONLY, out, ldo, grad_out, ldg, ctx, grad_feat, ldgf, grad_feat_lp, ldlp,
                        grad_attn_l, grad_attn_r, ws, ws_bytes, stream);
  Shape s;
  if ((rc = check_shape(heads, head_dim, dtype, s)) != MEGA_OK) return rc;
  if (!feat || !attn_l || !attn_r || !out || !grad_out || !ctx || !grad_feat || !grad_attn_l || !grad_attn_r || !ws)
    return fail(MEGA_ERR_INVALID_ARGUMENT, "null pointer");
  const int esz = dtype == MEGA_BF16 ? 2 : 4;
  if (ldf < s.D || ldo < s.D || ldg < s.D || ldgf != s.D || (ldf * esz) % 16 || (ldo * esz) % 16 ||
      (ldg * esz) % 16 || (ldgf * 4) % 16)
    return fail(MEGA_ERR_INVALID_ARGUMENT, "leading dimensions must be >= D (ldgf == D) and multiples of 16 bytes");
  if ((uint64_t)L->n * (uint64_t)std::max(ldf, ldg) >= (1ULL << 32))
    return fail(MEGA_ERR_UNSUPPORTED, "num_nodes * ld must be < 2^32 elements (32-bit row offsets)");
  if (grad_feat_lp && (ldlp < s.D || (ldlp * esz) % 16 || !al16(grad_feat_lp)))
    return fail(MEGA_ERR_INVALID_ARGUMENT, "grad_feat_lp: bad ld or alignment");
  if (!al16(feat) || !al16(out) || !al16(grad_out) || !al16(ctx) || !al16(grad_feat) || !al16(ws) ||
      !al16(attn_l) || !al16(attn_r))
    return fail(MEGA_ERR_INVALID_ARGUMENT, "pointers must be 16-byte aligned");
  const Part &P = L->parts[part];
  const DistWs dw = dist_ws(L, part, s);
  if (ws_bytes < dw.bwd_total) return fail(MEGA_ERR_OUT_OF_MEMORY, "bwd workspace too small (mega_gat_dist_workspace_bytes)");
  bool snd, rcv;
  phase_flags(flags, snd, rcv);
  const int64_t plane = L->n * s.H, b0 = P.row_begin, rows = P.row_end - P.row_begin;
  kern::BwdArgs a;
  a.L = P.dev;
  a.feat = feat; a.ldf = ldf; a.al = attn_l; a.ar = attn_r;
  a.H = s.H; a.F = s.F; a.D = s.D; a.slope = negative_slope;
  a.out = out; a.ldo = ldo; a.gout = grad_out; a.ldg = ldg;
  a.el = ctx; a.er = ctx + plane; a.lse = ctx + 2 * plane; a.dlt = ctx + 3 * plane; a.der = ctx + 4 * plane;
  a.gfeat = grad_feat; a.ldgf = ldgf; a.gfeat_lp = grad_feat_lp; a.ldlp = ldlp;
  const WsBwd w = ws_bwd(P.dev, s);
  char *wb = static_cast<char *>(ws);
  a.dz = reinterpret_cast<float *>(wb + w.dz);
  a.ws_bacc = reinterpret_cast<float *>(wb + w.bacc);
  a.ws_bder = reinterpret_cast<float *>(wb + w.bder);
  a.ws_dal = reinterpret_cast<double *>(wb + w.dal);
  a.ws_dar = reinterpret_cast<double *>(wb + w.dar);
  a.gal = grad_attn_l; a.gar = grad_attn_r;
  a.nb_dst = 0;
  a.lp_only = (flags & MEGA_BWD_LP_ONLY) && grad_feat_lp ? 1 : 0;
  a.lp_partial = 0;   // the exchange moves fp32 partials of grad_feat rows
  a.st_hint = st_hint_mode();
  a.ctr = nullptr;
  cudaStream_t st = (cudaStream_t)stream, cs = (cudaStream_t)comm_stream;
  // counters 0..2: the three source-phase launches of the SEND phase (zeroed there)
  int *ctrs = sched_dynamic() ? reinterpret_cast<int *>(wb + w.ctr) : nullptr;
  int npass = 0;
  // source-phase launches over a range of CSC items [i0, i1) and splits [s0, s1)
  auto src_range = [&](int32_t i0, int32_t i1, int32_t s0, int32_t s1, bool dlt) {
    kern::BwdArgs b = a;
    b.ctr = ctrs ? ctrs + npass++ : nullptr;
    b.L.bwd_items = P.dev.bwd_items + i0; b.L.n_bwd_items = std::max(0, i1 - i0); b.L.bchunk = nullptr;
    b.L.bwd_splits = P.dev.bwd_splits + 3 * s0; b.L.n_bwd_splits = std::max(0, s1 - s0);
    return dtype == MEGA_BF16 ? run_bwd<__nv_bfloat16>(b, s, MEGA_BWD_PHASE_SRC, st, dev, dlt)
                              : run_bwd<float>(b, s, MEGA_BWD_PHASE_SRC, st, dev, dlt);
  };
  // NEXT-1 halo: this rank's partials of the peers' rows its edges reference go back to their owners
  // (the forward's receive lists), the peers' partials of our rows arrive in send-list order
  const int k = (int)L->parts.size();
  const size_t rf = (size_t)s.D * 4, re = (size_t)s.H * 4;
  char *sf = wb + dw.b_sf, *se = wb + dw.b_se, *rfb = wb + dw.b_rf, *reb = wb + dw.b_re;
  std::vector<CommMsg> sends, recvs;
  for (int q = 0; q < k; ++q) {
    if (q == part) continue;
    const int64_t s0 = P.hrecv_off[q], sn = P.hrecv_off[q + 1] - s0, r0 = P.hsend_off[q], rn = P.hsend_off[q + 1] - r0;
    sends.push_back({q, 2, sf + s0 * rf, (size_t)sn * rf});
    sends.push_back({q, 3, se + s0 * re, (size_t)sn * re});
    recvs.push_back({q, 2, rfb + r0 * rf, (size_t)rn * rf});
    recvs.push_back({q, 3, reb + r0 * re, (size_t)rn * re});
  }
  const DevPart &D = P.dev;
  if (snd) {
    if (ctrs) {
      cudaError_t ce = cudaMemsetAsync(ctrs, 0, kCtrs * 4, st);
      if (ce != cudaSuccess) return fail(MEGA_ERR_CUDA, std::string("counter reset: ") + cudaGetErrorString(ce));
    }
    // Dlt, then the sources other ranks own (their partials travel while ours are computed)
    if ((rc = src_range(0, D.bwd_own0, 0, D.bsplit_own0, true)) != MEGA_OK) return rc;
    if ((rc = src_range(D.bwd_own1, D.n_bwd_items, D.bsplit_own1, D.n_bwd_splits, false)) != MEGA_OK) return rc;
    if ((rc = move_rows(grad_feat, ldgf * 4, D.hrecv_idx, sf, rf, nullptr, D.n_hrecv, (int)rf, st, dev)) != MEGA_OK) return rc;
    if ((rc = move_rows(ctx + 4 * plane, re, D.hrecv_idx, se, re, nullptr, D.n_hrecv, (int)re, st, dev)) != MEGA_OK) return rc;
    if ((rc = comm_exchange(comm, sends, recvs, st, cs, true, false)) != MEGA_OK) return rc;
    if ((rc = src_range(D.bwd_own0, D.bwd_own1, D.bsplit_own0, D.bsplit_own1, false)) != MEGA_OK) return rc;
  }
  if (rcv) {
    if ((rc = comm_exchange(comm, sends, recvs, st, cs, false, true)) != MEGA_OK) return rc;
    cudaError_t ce = cudaStreamWaitEvent(st, comm_done_event(comm), 0);
    if (ce != cudaSuccess) return fail(MEGA_ERR_CUDA, std::string("wait comm: ") + cudaGetErrorString(ce));
    if (k > 1 && rows > 0) {
      const int64_t nv = rows * (s.D / 4);
      const int blocks = (int)std::min<int64_t>((nv + 255) / 256, 4 * dev_info(dev).sms);
      kern::dist_combine_kernel<<<std::max(blocks, 1), 256, 0, st>>>(
          grad_feat, ldgf, ctx + 4 * plane, reinterpret_cast<const float *>(rfb), reinterpret_cast<const float *>(reb),
          D.hpos, k - 1, rows, b0, s.D, s.H);
      if ((rc = check_launch(st, "dist_combine_kernel")) != MEGA_OK) return rc;
    }
    rc = dtype == MEGA_BF16 ? run_bwd<__nv_bfloat16>(a, s, MEGA_BWD_PHASE_DST, st, dev)
                            : run_bwd<float>(a, s, MEGA_BWD_PHASE_DST, st, dev);
    if (rc != MEGA_OK) return rc;
  }
  return MEGA_OK;
}

}  // extern "C"
