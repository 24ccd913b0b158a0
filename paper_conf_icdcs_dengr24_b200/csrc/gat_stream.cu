// a3-a5, edge-streaming forward for wide rows (G = 32 lanes per row, i.e.
// feature rows of >= 512 bytes: arxiv, Reddit, products).  Two passes:
//
//   A. fwd_stats_kernel: per destination i and head h the softmax statistics
//      lse_i = m_i + log sum_e exp(s_e - m_i), s_e = LeakyReLU(el_i + er_j)
//      (PAPER.md:51-55 skeleton; R1-R3), then the normalised
//      weights alpha_e = exp(s_e - lse_i), written in CSR order (4H B per
//      edge).  Reads 4 B of index and 4H B of er per edge.  Rows longer than S
//      are split into work items whose partial (m, S) merge in fixed order
//      (fwd_stats_merge_kernel); their alpha come from fwd_alpha_split_kernel.
//   B. gat_fwd_agg_kernel: out_i = sum_e alpha_e Wh_j, a weighted SpMM.  The
//      edges are cut into tiles of whole rows (<= kTileEdges edges; a split
//      segment is a tile of its own and writes an fp32 partial that
//      gat_fwd_split_sum_kernel adds in segment order).  Warps take tiles
//      grid-stride, so the warps in flight work on neighbouring rows of the
//      (L2-blocked) order, and each warp streams its tiles as ONE pipeline:
//      source rows are moved by TMA bulk copies (cp.async.bulk, one row per
//      copy, up to 4 rows per mbarrier) into a per-warp shared-memory ring;
//      per-edge metadata (source, row, alpha) is loaded two 32-edge chunks
//      ahead, so the ring does not drain at row ends.
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <cstdlib>

#include "kern_common.cuh"
#include "mega_internal.h"

namespace mega {
namespace kern {

// ---------------------------------------------------------------- TMA / mbarrier
__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t *bar, unsigned count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t *bar, unsigned bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, unsigned bytes, uint64_t *bar, uint64_t pol) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(pol)
      : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *bar, unsigned parity) {
  uint32_t ok = 0;
  do {
    asm volatile(
        "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}\n"
        : "=r"(ok)
        : "r"(smem_u32(bar)), "r"(parity)
        : "memory");
  } while (!ok);
}

// ---------------------------------------------------------------- pass A
// G = 8 lanes per work item; every lane keeps a private online (m, S) over the
// edges e = e0 + gl, e0 + gl + 8, ... (two edges per step for memory-level
// parallelism), then the group combines them and (unsplit rows) writes alpha.
template <int HT>
__device__ __forceinline__ void store_alpha(float *p, const float (&v)[HT]) {
  if constexpr (HT == 1) {
    *p = v[0];
  } else if constexpr (HT == 2) {
    *reinterpret_cast<float2 *>(p) = make_float2(v[0], v[1]);
  } else {
#pragma unroll
    for (int q = 0; q < HT / 4; ++q)
      reinterpret_cast<float4 *>(p)[q] = make_float4(v[4 * q], v[4 * q + 1], v[4 * q + 2], v[4 * q + 3]);
  }
}

template <int HT, int G>
__device__ __forceinline__ void write_alpha(const FwdArgs &a, int e0, int e1, int gl, const float (&el)[HT],
                                            const float (&lse)[HT], uint64_t pol) {
  const uint32_t idm = a.L.id_mask;
  for (int e = e0 + gl; e < e1; e += G) {
    const uint32_t j = (uint32_t)ld_stream(a.L.src + e, pol) & idm;
    float r[HT], al[HT];
    load_h<HT>(a.er + (int64_t)j * HT, HT, r);
#pragma unroll
    for (int h = 0; h < HT; ++h) al[h] = fexp(leaky(el[h] + r[h], a.slope) - lse[h]);
    store_alpha<HT>(a.alpha + (int64_t)e * HT, al);
  }
}

template <int HT>
__global__ void __launch_bounds__(TPB) fwd_stats_kernel(const FwdArgs a, int esz) {
  constexpr int G = 8, GPW = 4;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, gl = lane % G, grp = lane / G;
  const unsigned gmask = 0xffu << (grp * G);
  const uint32_t idm = a.L.id_mask;
  const uint64_t pol = policy_first();
  const int64_t stride = (int64_t)gridDim.x * WPB * GPW;
  for (int64_t it = ((int64_t)blockIdx.x * WPB + w) * GPW + grp; it < a.L.n_fwd_items; it += stride) {
    const int4 item = a.L.fwd_items[it];
    const int64_t grow = a.L.row_begin + item.x;
    float el[HT], m[HT], l[HT];
    load_h<HT>(a.el + grow * HT, HT, el);
#pragma unroll
    for (int h = 0; h < HT; ++h) { m[h] = -INFINITY; l[h] = 0.f; }
    for (int e = item.y + gl; e < item.z; e += 2 * G) {
      const bool two = e + G < item.z;
      const uint32_t j0 = (uint32_t)ld_stream(a.L.src + e, pol) & idm;
      const uint32_t j1 = (uint32_t)ld_stream(a.L.src + (two ? e + G : e), pol) & idm;
      float r0[HT], r1[HT];
      load_h<HT>(a.er + (int64_t)j0 * HT, HT, r0);
      load_h<HT>(a.er + (int64_t)j1 * HT, HT, r1);
#pragma unroll
      for (int h = 0; h < HT; ++h) {
        const float s0 = leaky(el[h] + r0[h], a.slope);
        const float s1 = two ? leaky(el[h] + r1[h], a.slope) : -INFINITY;
        const float mn = fmaxf(m[h], fmaxf(s0, s1));
        l[h] = l[h] * fexp(m[h] - mn) + fexp(s0 - mn) + (two ? fexp(s1 - mn) : 0.f);
        m[h] = mn;
      }
    }
    float M[HT], L[HT];
#pragma unroll
    for (int h = 0; h < HT; ++h) {
      M[h] = gmax<G>(m[h], gmask);
      L[h] = gsum<G>(l[h] > 0.f ? l[h] * fexp(m[h] - M[h]) : 0.f, gmask);
    }
    if (item.w < 0) {
      float lse[HT];
#pragma unroll
      for (int h = 0; h < HT; ++h) lse[h] = L[h] > 0.f ? M[h] + flog(L[h]) : -INFINITY;
      for (int h = gl; h < HT; h += G) a.lse[grow * HT + h] = sel<HT>(lse, h);
      if (item.y == item.z) {  // no in-edges: out = 0 (R6)
        uint4 *orow = reinterpret_cast<uint4 *>(static_cast<char *>(a.out) + (int64_t)item.x * a.ldo * esz);
        for (int q = gl; q < a.D * esz / 16; q += G) orow[q] = make_uint4(0, 0, 0, 0);
      } else {
        write_alpha<HT, G>(a, item.y, item.z, gl, el, lse, pol);
      }
    } else {
      for (int h = gl; h < HT; h += G) {
        a.ws_m[(int64_t)item.w * HT + h] = sel<HT>(M, h);
        a.ws_l[(int64_t)item.w * HT + h] = sel<HT>(L, h);
      }
    }
  }
}

// lse of split rows: M = max m_k, L = sum l_k e^{m_k - M} in segment order.
__global__ void fwd_stats_merge_kernel(const FwdArgs a) {
  const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= (int64_t)a.L.n_fwd_splits * a.H) return;
  const int k = (int)(t / a.H), h = (int)(t % a.H);
  const int row = a.L.fwd_splits[3 * k], s0 = a.L.fwd_splits[3 * k + 1], ns = a.L.fwd_splits[3 * k + 2];
  float M = -INFINITY;
  for (int q = 0; q < ns; ++q) M = fmaxf(M, a.ws_m[(int64_t)(s0 + q) * a.H + h]);
  float L = 0.f;
  for (int q = 0; q < ns; ++q) {
    const float lq = a.ws_l[(int64_t)(s0 + q) * a.H + h];
    if (lq > 0.f) L += lq * fexp(a.ws_m[(int64_t)(s0 + q) * a.H + h] - M);
  }
  a.lse[(a.L.row_begin + row) * a.H + h] = L > 0.f ? M + flog(L) : -INFINITY;
}

// alpha of split rows (after the merge): one 32-lane group per segment item.
template <int HT>
__global__ void __launch_bounds__(TPB) fwd_alpha_split_kernel(const FwdArgs a) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const uint64_t pol = policy_first();
  for (int64_t it = (int64_t)blockIdx.x * WPB + w; it < a.L.n_fwd_items; it += (int64_t)gridDim.x * WPB) {
    const int4 item = a.L.fwd_items[it];
    if (item.w < 0) continue;
    const int64_t grow = a.L.row_begin + item.x;
    float el[HT], lse[HT];
    load_h<HT>(a.el + grow * HT, HT, el);
    load_h<HT>(a.lse + grow * HT, HT, lse);
    write_alpha<HT, 32>(a, item.y, item.z, lane, el, lse, pol);
  }
}

// ---------------------------------------------------------------- pass B
template <int V> struct AggCfg {
  static constexpr int RB = 32 * V * 16;                                       // bytes per row
  static constexpr int NQ = (12288 / (4 * RB)) < 2 ? 2 : (12288 / (4 * RB));  // ring quads per warp (4 rows each)
  static constexpr size_t SMEM = (size_t)WPB * NQ * 4 * RB + (size_t)WPB * NQ * 8;
};

template <typename T, int V, int HT>
__global__ void __launch_bounds__(TPB, 2) gat_fwd_agg_kernel(const FwdArgs a) {
  constexpr int EPV = Tr<T>::EPV, FF = 32 * V * EPV / HT, RB = AggCfg<V>::RB, NQ = AggCfg<V>::NQ, RV = RB / 16;
  extern __shared__ __align__(128) uint4 dyn[];
  __shared__ int s_j[WPB][3][32], s_r[WPB][3][32];
  __shared__ __align__(16) float s_a[WPB][3][32][HT];
  __shared__ int s_len[WPB][3], s_dst[WPB][3];  // chunk length; flush destination (-2 = continue tile, else slot|-1)
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  uint4 *ring = dyn + (size_t)w * NQ * 4 * RV;
  uint64_t *bars = reinterpret_cast<uint64_t *>(dyn + (size_t)WPB * NQ * 4 * RV) + w * NQ;
  const uint32_t idm = a.L.id_mask;
  const int hot_cls = a.hot_cls;
  const uint64_t pol_hot = row_policy_hot(a.pol_mode), pol_row = row_policy_cold(a.pol_mode), pol_cold = policy_first();
  const char *featb = static_cast<const char *>(a.feat);
  const int64_t rowstride = a.ldf * (int64_t)sizeof(T);
  const int ntiles = a.L.n_ftiles;
  const int W = gridDim.x * WPB, gw = blockIdx.x * WPB + w;
  if (gw >= ntiles) return;
  if (lane < NQ) mbar_init(&bars[lane], 1);
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  __syncwarp();
  const float *sa_v[V];
#pragma unroll
  for (int v = 0; v < V; ++v) sa_v[v] = &s_a[w][0][0][((v * 32 + lane) * EPV) / FF];

  // ---- producer: chunks of <= 32 edges of this warp's tiles, in order ----
  int pt = gw, pe = 0, pend = 0, pslot = -1;  // current producer tile
  bool pnew = true;
  if (pt < ntiles) {
    const int4 t = a.L.ftiles[pt];
    pe = t.x; pend = t.y; pslot = t.z;
  }
  // one chunk of metadata in registers: source, row, alpha of lane's edge; uniform len / dst
  int qj = 0, qr = 0, qlen = 0, qdst = -2;
  float qa[HT];
  auto produce = [&]() {  // load the next chunk into the register set (qlen = 0: none left)
    if (pt >= ntiles) { qlen = 0; return; }
    qlen = min(32, pend - pe);
    qdst = pnew ? pslot : -2;
    const int e = pe + min(lane, qlen - 1);
    qj = ld_stream(a.L.src + e, pol_cold);
    qr = ld_stream(a.L.erow + e, pol_cold);
    load_h_v<HT>(a.alpha + (int64_t)e * HT, HT, qa);
    pe += qlen;
    pnew = false;
    if (pe >= pend) {
      pt += W;
      pnew = true;
      if (pt < ntiles) {
        const int4 t = a.L.ftiles[pt];
        pe = t.x; pend = t.y; pslot = t.z;
      }
    }
  };
  auto store = [&](int b) {  // register chunk -> shared buffer b
    s_j[w][b][lane] = qj;
    s_r[w][b][lane] = qr;
#pragma unroll
    for (int h = 0; h < HT; ++h) s_a[w][b][lane][h] = lane < qlen ? qa[h] : 0.f;
    if (lane == 0) { s_len[w][b] = qlen; s_dst[w][b] = qdst; }
  };
  // ---- ring: quads of <= 4 rows of one chunk; issue cursor (ib, il) runs ahead of consumption ----
  int ib = 0, il = 0, iq = 0, cq = 0;  // issue chunk buffer / lane; quads issued / consumed
  int avail = 0;                        // chunks with metadata in shared memory, ahead of the issue cursor incl.
  auto issue_quads = [&]() {
    while (iq - cq < NQ && avail > 0) {
      const int len = s_len[w][ib];
      const int cnt = min(4, len - il);
      const int q = iq % NQ;
      if (lane == 0) {
        mbar_expect_tx(&bars[q], cnt * RB);
        for (int u = 0; u < cnt; ++u) {
          const uint32_t jj = (uint32_t)s_j[w][ib][il + u];
          const uint64_t pol = (int)(jj >> 26) >= hot_cls ? pol_hot : pol_row;
          bulk_g2s(ring + (q * 4 + u) * RV, featb + (int64_t)(jj & idm) * rowstride, RB, &bars[q], pol);
        }
      }
      ++iq;
      il += cnt;
      if (il >= len) { il = 0; ib = ib == 2 ? 0 : ib + 1; --avail; }
    }
  };

  // prologue: chunk 0 -> smem, chunk 1 -> registers
  produce();
  store(0);
  produce();
  __syncwarp();
  avail = 1;
  issue_quads();

  float acc[V][EPV];
#pragma unroll
  for (int v = 0; v < V; ++v)
#pragma unroll
    for (int k = 0; k < EPV; ++k) acc[v][k] = 0.f;
  int cur = -1, cur_dst = -1;
  auto flush = [&]() {
    if (cur_dst >= 0) {
      float *dst = a.ws_acc + (int64_t)cur_dst * a.D;
#pragma unroll
      for (int v = 0; v < V; ++v)
#pragma unroll
        for (int k = 0; k < EPV; k += 4)
          *reinterpret_cast<float4 *>(dst + (v * 32 + lane) * EPV + k) =
              make_float4(acc[v][k], acc[v][k + 1], acc[v][k + 2], acc[v][k + 3]);
    } else {
      T *orow = static_cast<T *>(a.out) + (int64_t)cur * a.ldo + lane * EPV;
#pragma unroll
      for (int v = 0; v < V; ++v) st16(orow + v * 32 * EPV, pack(acc[v], T()));
    }
#pragma unroll
    for (int v = 0; v < V; ++v)
#pragma unroll
      for (int k = 0; k < EPV; ++k) acc[v][k] = 0.f;
  };

  int cb = 0;  // consumption chunk buffer
  for (;;) {
    const int len = s_len[w][cb];
    if (len == 0) break;
    const int dst = s_dst[w][cb];
    // the chunk after next enters shared memory; the one after that is loaded
    if (qlen > 0) {
      store(cb == 2 ? 0 : cb + 1 == 2 ? 2 : cb + 1);
      produce();
      ++avail;
    } else {
      if (lane == 0) s_len[w][cb == 2 ? 0 : cb + 1] = 0;
    }
    __syncwarp();
    issue_quads();
    if (dst != -2) {  // first chunk of a tile: close the previous tile's row
      if (cur >= 0) flush();
      cur = -1;
      cur_dst = dst;
    }
    const int *sr = s_r[w][cb];
    for (int l0 = 0; l0 < len; l0 += 4) {
      const int q = cq % NQ;
      mbar_wait(&bars[q], (unsigned)(cq / NQ) & 1u);
      const int cnt = min(4, len - l0);
      for (int u = 0; u < cnt; ++u) {
        const int l = l0 + u;
        const int r = sr[l];
        if (r != cur) {
          if (cur >= 0) flush();
          cur = r;
        }
        const uint4 *row = ring + (q * 4 + u) * RV;
#pragma unroll
        for (int v = 0; v < V; ++v) {
          const float pw = sa_v[v][(cb * 32 + l) * HT];
          float x[EPV];
          unpack(row[v * 32 + lane], x, T());
#pragma unroll
          for (int k = 0; k < EPV; k += 2) ffma2s(acc[v][k], acc[v][k + 1], x[k], x[k + 1], pw);
        }
      }
      __syncwarp();
      ++cq;
      issue_quads();
    }
    cb = cb == 2 ? 0 : cb + 1;
  }
  if (cur >= 0) flush();
}

// out of split rows: the sum of their segments' fp32 partials, in segment order.
template <typename T, int V>
__global__ void __launch_bounds__(TPB) gat_fwd_split_sum_kernel(const FwdArgs a) {
  constexpr int EPV = Tr<T>::EPV;
  const int lane = threadIdx.x & 31;
  const int64_t k = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  if (k >= a.L.n_fwd_splits) return;
  const int row = a.L.fwd_splits[3 * k], s0 = a.L.fwd_splits[3 * k + 1], ns = a.L.fwd_splits[3 * k + 2];
  float acc[V][EPV];
#pragma unroll
  for (int v = 0; v < V; ++v)
#pragma unroll
    for (int q = 0; q < EPV; ++q) acc[v][q] = 0.f;
  for (int s = 0; s < ns; ++s) {
    const float *p = a.ws_acc + (int64_t)(s0 + s) * a.D;
#pragma unroll
    for (int v = 0; v < V; ++v)
#pragma unroll
      for (int q = 0; q < EPV; ++q) acc[v][q] += p[(v * 32 + lane) * EPV + q];
  }
  T *orow = static_cast<T *>(a.out) + (int64_t)row * a.ldo + lane * EPV;
#pragma unroll
  for (int v = 0; v < V; ++v) st16(orow + v * 32 * EPV, pack(acc[v], T()));
}

}  // namespace kern

// ---------------------------------------------------------------- host
namespace {
using namespace kern;

template <typename T, int V, int HT>
mega_status launch_stream(const FwdArgs &a0, cudaStream_t st, int sms) {
  FwdArgs a = a0;
  constexpr int esz = sizeof(T);
  mega_status rc = MEGA_OK;
  auto chk = [&](const char *what) {
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) rc = fail(MEGA_ERR_CUDA, std::string(what) + ": " + cudaGetErrorString(e));
    return rc == MEGA_OK;
  };
  if (a.L.n_fwd_items > 0) {
    const int64_t groups = a.L.n_fwd_items;
    const int grid = (int)std::max<int64_t>(1, std::min<int64_t>((groups + WPB * 4 - 1) / (WPB * 4), (int64_t)sms * 8));
    fwd_stats_kernel<HT><<<grid, TPB, 0, st>>>(a, esz);
    if (!chk("fwd_stats_kernel")) return rc;
  }
  if (a.L.n_fwd_splits > 0) {
    const int64_t t = (int64_t)a.L.n_fwd_splits * a.H;
    fwd_stats_merge_kernel<<<(int)((t + 255) / 256), 256, 0, st>>>(a);
    if (!chk("fwd_stats_merge_kernel")) return rc;
    fwd_alpha_split_kernel<HT><<<sms * 4, TPB, 0, st>>>(a);
    if (!chk("fwd_alpha_split_kernel")) return rc;
  }
  if (a.L.n_ftiles == 0) return MEGA_OK;
  auto k = gat_fwd_agg_kernel<T, V, HT>;
  constexpr size_t smem = AggCfg<V>::SMEM;
  cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  int per_sm = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k, TPB, smem);
  per_sm = std::max(1, per_sm);
  int64_t grid = (int64_t)sms * per_sm;
  grid = std::min<int64_t>(grid, ((int64_t)a.L.n_ftiles + WPB - 1) / WPB);
  k<<<(int)std::max<int64_t>(1, grid), TPB, smem, st>>>(a);
  if (!chk("gat_fwd_agg_kernel")) return rc;
  if (a.L.n_fwd_splits > 0) {
    gat_fwd_split_sum_kernel<T, V><<<(int)(((int64_t)a.L.n_fwd_splits * 32 + TPB - 1) / TPB), TPB, 0, st>>>(a);
    chk("gat_fwd_split_sum_kernel");
  }
  return rc;
}
}  // namespace

mega_status run_fwd_stream(const kern::FwdArgs &a, int nv, int H, bool bf16, cudaStream_t st, int sms) {
  // wide rows only: nv = row bytes / 16 in {32, 64, 128, 256} -> V = nv / 32
  auto go = [&](auto tag) -> mega_status {
    using T = decltype(tag);
    auto byh = [&](auto vtag) -> mega_status {
      constexpr int V = decltype(vtag)::value;
      switch (H) {
        case 1: return launch_stream<T, V, 1>(a, st, sms);
        case 2: return launch_stream<T, V, 2>(a, st, sms);
        case 4: return launch_stream<T, V, 4>(a, st, sms);
        default: return launch_stream<T, V, 8>(a, st, sms);
      }
    };
    switch (nv) {
      case 32: return byh(std::integral_constant<int, 1>());
      case 64: return byh(std::integral_constant<int, 2>());
      case 128: return byh(std::integral_constant<int, 4>());
      case 256: return byh(std::integral_constant<int, 8>());
      default: return fail(MEGA_ERR_UNSUPPORTED, "edge-streaming forward: unsupported row width");
    }
  };
  return bf16 ? go(__nv_bfloat16()) : go(float());
}

}  // namespace mega
