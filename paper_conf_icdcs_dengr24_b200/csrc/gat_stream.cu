// a3-a5, edge-streaming forward for wide rows (G = 32 lanes per row, i.e.
// feature rows of >= 512 bytes: arxiv, Reddit, products).  Two passes:
//
//   A. fwd_stats_kernel: per destination i and head h the softmax statistics
//      lse_i = m_i + log sum_e exp(s_e - m_i), s_e = LeakyReLU(el_i + er_j)
//      (PAPER.md:51-55 skeleton; R1-R3).  Reads 4 B of index and
//      4H B of er per edge; rows longer than S are split into work items whose
//      partial (m, S) merge in fixed order (fwd_stats_merge_kernel).
//   B. gat_fwd_agg_kernel: out_i = sum_e alpha_e Wh_j with
//      alpha_e = exp(s_e - lse_i), a weighted SpMM.  Because alpha is already
//      normalised, partial sums of a row simply add: the part's edges are cut
//      into W equal contiguous ranges, one per warp (perfect balance for any
//      degree distribution), and each warp streams its range as ONE pipeline
//      across row boundaries.  Source rows are moved by TMA bulk copies
//      (cp.async.bulk, one 16-byte-aligned row per copy, completion on a
//      per-slot mbarrier) into a per-warp shared-memory ring of R rows, so R
//      rows stay in flight without holding registers and the pipeline never
//      drains at a row end.  Rows cut by a range boundary write fp32 partials
//      that gat_fwd_agg_fix_kernel adds in warp order (deterministic, no
//      atomics).  Per-edge metadata (source id, row, alpha) is prepared one
//      32-edge chunk ahead in a 3-deep shared ring.
#include <cuda_bf16.h>
#include <cuda_runtime.h>

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
// parallelism), then the group combines them.
template <int HT>
__global__ void __launch_bounds__(TPB) fwd_stats_kernel(const FwdArgs a, int esz) {
  constexpr int G = 8, GPW = 4;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, gl = lane % G, grp = lane / G;
  const unsigned gmask = 0xffu << (grp * G);
  const int H = a.H;
  const uint32_t idm = a.L.id_mask;
  const uint64_t pol = policy_first();
  const int64_t stride = (int64_t)gridDim.x * WPB * GPW;
  for (int64_t it = ((int64_t)blockIdx.x * WPB + w) * GPW + grp; it < a.L.n_fwd_items; it += stride) {
    const int4 item = a.L.fwd_items[it];
    const int64_t grow = a.L.row_begin + item.x;
    float el[HT], m[HT], l[HT];
    load_h<HT>(a.el + grow * H, H, el);
#pragma unroll
    for (int h = 0; h < HT; ++h) { m[h] = -INFINITY; l[h] = 0.f; }
    for (int e = item.y + gl; e < item.z; e += 2 * G) {
      const bool two = e + G < item.z;
      const uint32_t j0 = (uint32_t)ld_stream(a.L.src + e, pol) & idm;
      const uint32_t j1 = (uint32_t)ld_stream(a.L.src + (two ? e + G : e), pol) & idm;
      float r0[HT], r1[HT];
      load_h<HT>(a.er + (int64_t)j0 * H, H, r0);
      load_h<HT>(a.er + (int64_t)j1 * H, H, r1);
#pragma unroll
      for (int h = 0; h < HT; ++h) {
        if (h >= H) continue;
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
      for (int h = gl; h < H; h += G) {
        const float Lh = sel<HT>(L, h);
        a.lse[grow * H + h] = Lh > 0.f ? sel<HT>(M, h) + flog(Lh) : -INFINITY;
      }
      if (item.y == item.z) {  // no in-edges: out = 0 (R6)
        uint4 *orow = reinterpret_cast<uint4 *>(static_cast<char *>(a.out) + (int64_t)item.x * a.ldo * esz);
        for (int q = gl; q < a.D * esz / 16; q += G) orow[q] = make_uint4(0, 0, 0, 0);
      }
    } else {
      for (int h = gl; h < H; h += G) {
        a.ws_m[(int64_t)item.w * H + h] = sel<HT>(M, h);
        a.ws_l[(int64_t)item.w * H + h] = sel<HT>(L, h);
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

// ---------------------------------------------------------------- pass B
template <int V> struct AggCfg {
  static constexpr int RB = 32 * V * 16;                                   // bytes per row
  static constexpr int R = (10240 / RB) > 32 ? 32 : ((10240 / RB) < 2 ? 2 : 10240 / RB);  // ring rows per warp
  static constexpr size_t SMEM = (size_t)WPB * R * RB + (size_t)WPB * R * 8;
};

template <typename T, int V, int HT>
__global__ void __launch_bounds__(TPB, 2) gat_fwd_agg_kernel(const FwdArgs a) {
  constexpr int EPV = Tr<T>::EPV, FF = 32 * V * EPV / HT, RB = AggCfg<V>::RB, R = AggCfg<V>::R, RV = RB / 16;
  static_assert(R <= 32, "ring deeper than a metadata chunk");
  extern __shared__ __align__(128) uint4 dyn[];
  __shared__ int s_j[WPB][3][32], s_r[WPB][3][32];
  __shared__ float s_a[WPB][3][32][HT];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  uint4 *ring = dyn + (size_t)w * R * RV;
  uint64_t *bars = reinterpret_cast<uint64_t *>(dyn + (size_t)WPB * R * RV) + w * R;
  const int H = a.H;
  const uint32_t idm = a.L.id_mask;
  const int hot_cls = a.hot_cls;
  const uint64_t pol_hot = policy_last(), pol_cold = policy_first();
  const char *featb = static_cast<const char *>(a.feat);
  const int64_t rowstride = a.ldf * (int64_t)sizeof(T);
  int hv[V];
#pragma unroll
  for (int v = 0; v < V; ++v) hv[v] = ((v * 32 + lane) * EPV) / FF;

  const int64_t W = (int64_t)gridDim.x * WPB, gw = (int64_t)blockIdx.x * WPB + w, E = a.L.edges;
  const int64_t E0 = gw * E / W, E1 = (gw + 1) * E / W;
  const int n = (int)(E1 - E0);
  if (n <= 0) return;
  if (lane < R) mbar_init(&bars[lane], 1);
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  __syncwarp();

  auto ld_idx = [&](int c, int &j, int &r) {
    const int64_t q = E0 + min(c * 32 + lane, n - 1);
    j = ld_stream(a.L.src + q, pol_cold);
    r = ld_stream(a.L.erow + q, pol_cold);
  };
  auto ld_side = [&](int j, int r, float (&er)[HT], float (&el)[HT], float (&ls)[HT]) {
    load_h<HT>(a.er + (int64_t)((uint32_t)j & idm) * H, H, er);
    load_h<HT>(a.el + (a.L.row_begin + r) * H, H, el);
    load_h<HT>(a.lse + (a.L.row_begin + r) * H, H, ls);
  };
  auto put_alpha = [&](int c, const float (&er)[HT], const float (&el)[HT], const float (&ls)[HT]) {
    const bool valid = c * 32 + lane < n;
#pragma unroll
    for (int h = 0; h < HT; ++h) s_a[w][c % 3][lane][h] = valid && h < H ? fexp(leaky(el[h] + er[h], a.slope) - ls[h]) : 0.f;
  };
  auto issue = [&](int p, uint32_t jj) {  // position p of this warp's stream -> ring slot p % R
    const int slot = p % R;
    const uint64_t pol = (int)(jj >> 26) >= hot_cls ? pol_hot : pol_cold;
    mbar_expect_tx(&bars[slot], RB);
    bulk_g2s(ring + slot * RV, featb + (int64_t)(jj & idm) * rowstride, RB, &bars[slot], pol);
  };

  // prologue: chunk 0 metadata, chunk 1 indices, ring fill
  int nj = 0, nr = 0;
  {
    int j0, r0;
    ld_idx(0, j0, r0);
    if (n > 32) ld_idx(1, nj, nr);
    s_j[w][0][lane] = j0;
    s_r[w][0][lane] = r0;
    float er[HT], el[HT], ls[HT];
    ld_side(j0, r0, er, el, ls);
    put_alpha(0, er, el, ls);
    __syncwarp();
    if (lane < R && lane < n) issue(lane, (uint32_t)j0);
  }
  const int r_first = s_r[w][0][0];
  const int r_last = __ldg(a.L.erow + E1 - 1);
  const bool first_partial = E0 > __ldg(a.L.indptr + r_first);
  const bool last_partial = __ldg(a.L.indptr + r_last + 1) > E1;

  float acc[V][EPV];
#pragma unroll
  for (int v = 0; v < V; ++v)
#pragma unroll
    for (int k = 0; k < EPV; ++k) acc[v][k] = 0.f;
  int cur = -1;
  auto flush = [&](int r) {
    if ((r == r_first && first_partial) || (r == r_last && last_partial)) {
      float *dst = a.ws_part + (2 * gw + ((r == r_first && first_partial) ? 0 : 1)) * (int64_t)a.D;
#pragma unroll
      for (int v = 0; v < V; ++v)
#pragma unroll
        for (int k = 0; k < EPV; k += 4)
          *reinterpret_cast<float4 *>(dst + (v * 32 + lane) * EPV + k) =
              make_float4(acc[v][k], acc[v][k + 1], acc[v][k + 2], acc[v][k + 3]);
    } else {
      T *orow = static_cast<T *>(a.out) + (int64_t)r * a.ldo + lane * EPV;
#pragma unroll
      for (int v = 0; v < V; ++v) st16(orow + v * 32 * EPV, pack(acc[v], T()));
    }
  };

  float ern[HT], eln[HT], lsn[HT];
#pragma unroll
  for (int h = 0; h < HT; ++h) ern[h] = eln[h] = lsn[h] = 0.f;
  for (int p = 0; p < n; ++p) {
    const int c = p >> 5, l = p & 31, buf = c % 3;
    const bool has_next = (c + 1) * 32 < n;
    if (l == 0) {
      if (has_next) {
        s_j[w][(c + 1) % 3][lane] = nj;
        s_r[w][(c + 1) % 3][lane] = nr;
        ld_side(nj, nr, ern, eln, lsn);
      }
      if ((c + 2) * 32 < n) ld_idx(c + 2, nj, nr);
      __syncwarp();
    }
    if (l == 16 && has_next) {
      put_alpha(c + 1, ern, eln, lsn);
      __syncwarp();
    }
    const int r = s_r[w][buf][l];
    if (r != cur) {
      if (cur >= 0) flush(cur);
      cur = r;
#pragma unroll
      for (int v = 0; v < V; ++v)
#pragma unroll
        for (int k = 0; k < EPV; ++k) acc[v][k] = 0.f;
    }
    const int slot = p % R;
    mbar_wait(&bars[slot], (unsigned)(p / R) & 1u);
    const uint4 *row = ring + slot * RV;
#pragma unroll
    for (int v = 0; v < V; ++v) {
      const float pw = s_a[w][buf][l][hv[v]];
      float x[EPV];
      unpack(row[v * 32 + lane], x, T());
#pragma unroll
      for (int k = 0; k < EPV; k += 2) ffma2s(acc[v][k], acc[v][k + 1], x[k], x[k + 1], pw);
    }
    __syncwarp();
    const int q = p + R;
    if (lane == 0 && q < n) issue(q, (uint32_t)s_j[w][(q >> 5) % 3][q & 31]);
  }
  if (cur >= 0) flush(cur);
}

// Rows cut by warp-range boundaries: boundary g handles row r when it is the
// first boundary strictly inside r; out_r = partial(g-1, last) + sum over the
// following non-empty warps v whose range starts inside r of partial(v, first).
template <typename T, int V>
__global__ void __launch_bounds__(TPB) gat_fwd_agg_fix_kernel(const FwdArgs a, int64_t W) {
  constexpr int EPV = Tr<T>::EPV;
  const int lane = threadIdx.x & 31;
  const int64_t g = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t E = a.L.edges;
  if (g < 1 || g >= W) return;
  const int64_t eg = g * E / W, ep = (g - 1) * E / W;
  if (eg >= E) return;
  const int r = a.L.erow[eg];
  const int64_t ra = a.L.indptr[r], rb = a.L.indptr[r + 1];
  if (!(ra < eg) || ep > ra) return;
  float acc[V][EPV];
  const float *p = a.ws_part + (2 * (g - 1) + 1) * (int64_t)a.D;
#pragma unroll
  for (int v = 0; v < V; ++v)
#pragma unroll
    for (int k = 0; k < EPV; ++k) acc[v][k] = p[(v * 32 + lane) * EPV + k];
  for (int64_t vv = g; vv < W; ++vv) {
    const int64_t s0 = vv * E / W, s1 = (vv + 1) * E / W;
    if (s0 >= rb) break;
    if (s1 == s0) continue;
    const float *q = a.ws_part + (2 * vv) * (int64_t)a.D;
#pragma unroll
    for (int v = 0; v < V; ++v)
#pragma unroll
      for (int k = 0; k < EPV; ++k) acc[v][k] += q[(v * 32 + lane) * EPV + k];
  }
  T *orow = static_cast<T *>(a.out) + (int64_t)r * a.ldo + lane * EPV;
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
  }
  if (a.L.edges == 0) return MEGA_OK;
  auto k = gat_fwd_agg_kernel<T, V, HT>;
  constexpr size_t smem = AggCfg<V>::SMEM;
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    attr = true;
  }
  int per_sm = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k, TPB, smem);
  per_sm = std::max(1, per_sm);
  int64_t grid = (int64_t)sms * per_sm;
  grid = std::min<int64_t>(grid, std::max<int64_t>(1, (a.L.edges + WPB * 32 - 1) / (WPB * 32)));
  grid = std::min<int64_t>(grid, kStreamMaxWarps / WPB);
  k<<<(int)grid, TPB, smem, st>>>(a);
  if (!chk("gat_fwd_agg_kernel")) return rc;
  const int64_t W = grid * WPB;
  if (W > 1) {
    gat_fwd_agg_fix_kernel<T, V><<<(int)((W * 32 + TPB - 1) / TPB), TPB, 0, st>>>(a, W);
    chk("gat_fwd_agg_fix_kernel");
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
