// a2 / a9: the dense node projection and its backward on the 5th-generation
// tensor cores — the one real contraction of the path (north_star: tensor
// cores only here; PAPER.md:55 neural operator, PAPER.md:142 sgemm).
//
//   fwd  Wh[N,D] = X[N,K] W[K,D]           + epilogue el = Wh.a_l, er = Wh.a_r (per head)
//   dX   dX[N,K] = dWh[N,D] W^T
//   dW   dW[K,D] = X^T dWh                  (split over N, fixed-order reduction)
//
// One CTA computes a 128 x BN output tile with tcgen05.mma (kind::f16: bf16
// operands, fp32 accumulator in TMEM), operands staged in shared memory by TMA
// (cp.async.bulk.tensor, 128-byte swizzle) through an mbarrier ring of STAGES
// slots.  128 threads: lane 0 of warp 0 is the TMA producer, lane 0 of warp 1
// issues the MMAs (one thread per CTA, as tcgen05 requires); then all four
// warps drain TMEM with tcgen05.ld (warp w owns TMEM lanes = tile rows
// 32w..32w+31, one row per thread) for the epilogue.  Several CTAs share an SM
// (<= 256 TMEM columns and ~100 KB of shared memory each), so one CTA's
// epilogue overlaps another's main loop.
//
// Operand majors (UMMA descriptors, SWIZZLE_128B canonical layouts):
//   fwd: A = X   K-major (rows of X contiguous in K),  B = W   MN-major (W[k][n], n contiguous)
//   dX : A = dWh K-major,                              B = W   K-major  (W[n=k_in][k=d])
//   dW : A = X   MN-major (X[k=row][m=k_in]),          B = dWh MN-major (dWh[k=row][n=d])
// K-major SW128 atom: 8 rows x 128 B (64 bf16 of K), 8-row groups 1024 B apart
// (SBO); the k-th UMMA_K = 16 slice starts 32 B further.  MN-major SW128 atom:
// 8 k-rows x 128 B (64 bf16 of M/N); 64-wide M/N groups LBO apart (one TMA
// box = 64 k-rows x 128 B = 8 KB), 8-k-row groups 1024 B apart (SBO); the
// k-th UMMA_K slice starts 16 rows x 128 B = 2 KB further.
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <mutex>

#include "mega_internal.h"

namespace mega {
namespace umma {

constexpr int BM = 128, BK = 64, THREADS = 128;
enum Mode { FWD = 0, DX = 1, DW = 2 };

struct Args {
  int64_t M;        // output rows (fwd/dX: N; dW: K_in)
  int Nc;           // output columns (fwd: D; dX: K_in; dW: D)
  int64_t kb_total; // 64-wide K blocks of the whole reduction
  int64_t kb_split; // K blocks per CTA along z (dW split; else = kb_total)
  void *out;        // fwd / dX: bf16 [M][ldo]; dW: fp32 partials [z][Mpad][Nc]
  int64_t ldo;
  int64_t mpad;     // dW: rows per partial slab
  // fwd epilogue: el/er into the ctx planes
  float *el, *er;
  const float *al, *ar;
  int H, F;
  int64_t ctx_row0;
  int ntiles;       // fwd / dX: column tiles (grid.x = row tiles * ntiles)
};

// ------------------------------------------------------------------ PTX helpers
__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint32_t bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
  asm volatile(
      "{\n"
      ".reg .pred P1;\n"
      "WAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
      "@P1 bra DONE_%=;\n"
      "bra WAIT_%=;\n"
      "DONE_%=:\n"
      "}\n" ::"r"(bar),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void tma_load_2d(uint32_t dst, const CUtensorMap *map, int32_t x, int32_t y, uint32_t bar) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::"r"(dst),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(x), "r"(y), "r"(bar)
      : "memory");
}
// shared -> global tensor store (bulk group); the source must stay valid until the read completes
__device__ __forceinline__ void tma_store_2d(const CUtensorMap *map, uint32_t src, int32_t x, int32_t y) {
  asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%1, %2}], [%3];" ::"l"(
                   reinterpret_cast<uint64_t>(map)),
               "r"(x), "r"(y), "r"(src)
               : "memory");
}
// TMA prefetch of a 2-D box into L2 (no shared memory, no completion tracking)
__device__ __forceinline__ void tma_prefetch_2d(const CUtensorMap *map, int32_t x, int32_t y) {
  asm volatile("cp.async.bulk.prefetch.tensor.2d.L2.global.tile [%0, {%1, %2}];" ::"l"(reinterpret_cast<uint64_t>(map)),
               "r"(x), "r"(y)
               : "memory");
}
__device__ __forceinline__ void prefetch_tmap(const CUtensorMap *map) {
  asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(map)) : "memory");
}
// shared-memory matrix descriptor, SWIZZLE_128B, sm_100 version bits
__device__ __forceinline__ uint64_t sdesc(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
  return (uint64_t)((saddr >> 4) & 0x3FFFu) | ((uint64_t)((lbo >> 4) & 0x3FFFu) << 16) |
         ((uint64_t)((sbo >> 4) & 0x3FFFu) << 32) | ((uint64_t)1 << 46) | ((uint64_t)2 << 61);
}
__device__ __forceinline__ void umma_f16(uint32_t tmem_d, uint64_t a, uint64_t b, uint32_t idesc, uint32_t accum) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "setp.ne.b32 p, %4, 0;\n"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n"
      "}\n" ::"r"(tmem_d),
      "l"(a), "l"(b), "r"(idesc), "r"(accum)
      : "memory");
}
__device__ __forceinline__ void umma_commit(uint32_t bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }

// 32 consecutive fp32 TMEM columns of this thread's lane
__device__ __forceinline__ void tmem_ld32(uint32_t taddr, uint32_t (&r)[32]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, %15, "
      "%16, %17, %18, %19, %20, %21, %22, %23, %24, %25, %26, %27, %28, %29, %30, %31}, [%32];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]), "=r"(r[8]),
        "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]), "=r"(r[16]),
        "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]), "=r"(r[24]),
        "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
      : "r"(taddr));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}
// packed fp32x2 FMA (sm_100 FFMA2): d{0,1} += a{0,1} * c{0,1}
__device__ __forceinline__ void ffma2(float &d0, float &d1, float a0, float a1, float c0, float c1) {
  unsigned long long D, A, C;
  asm("mov.b64 %0, {%1, %2};" : "=l"(A) : "f"(a0), "f"(a1));
  asm("mov.b64 %0, {%1, %2};" : "=l"(C) : "f"(c0), "f"(c1));
  asm("mov.b64 %0, {%1, %2};" : "=l"(D) : "f"(d0), "f"(d1));
  asm("fma.rn.f32x2 %0, %1, %2, %0;" : "+l"(D) : "l"(A), "l"(C));
  asm("mov.b64 {%0, %1}, %2;" : "=f"(d0), "=f"(d1) : "l"(D));
}
__device__ __forceinline__ uint32_t bf2(float a, float b) {
  __nv_bfloat162 t = __floats2bfloat162_rn(a, b);
  return *reinterpret_cast<uint32_t *>(&t);
}

template <int BN> struct Tiles {
  static constexpr int A_BYTES = BM * BK * 2;          // 16 KB
  static constexpr int B_BYTES = BN * BK * 2;
  static constexpr int STAGE = A_BYTES + B_BYTES;
  static constexpr int STAGES = STAGE >= 40 * 1024 ? 2 : (STAGE >= 28 * 1024 ? 3 : 4);
  static constexpr int TMEM_COLS = BN <= 32 ? 32 : BN <= 64 ? 64 : BN <= 128 ? 128 : 256;
  static constexpr size_t SMEM = 1024 + (size_t)STAGES * STAGE + 256 + 2 * BN * 4;
};

// MODE: FWD/DX/DW.  BN: tile columns (<= 256, multiple of 16; a multiple of 64
// when B is MN-major).  FH: fwd only, min(head_dim, 32) (heads per 32-column chunk).
template <int MODE, int BN, int FH>
__global__ void __launch_bounds__(THREADS) umma_gemm_kernel(const __grid_constant__ CUtensorMap tmA,
                                                            const __grid_constant__ CUtensorMap tmB,
                                                            const __grid_constant__ CUtensorMap tmO, const Args g) {
  using TL = Tiles<BN>;
  constexpr int STAGES = TL::STAGES;
  constexpr bool A_MN = MODE == DW, B_MN = MODE != DX;
  extern __shared__ uint8_t smem_raw[];
  uint8_t *smem = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~(uintptr_t)1023);
  uint64_t *bars = reinterpret_cast<uint64_t *>(smem + STAGES * TL::STAGE);   // full[S], empty[S], done
  uint32_t *tslot = reinterpret_cast<uint32_t *>(bars + 2 * STAGES + 1);
  float *s_al = reinterpret_cast<float *>(smem + STAGES * TL::STAGE + 256);
  float *s_ar = s_al + BN;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  // fwd / dX: one linear grid with the column tile fastest, so the CTAs that share a row tile of A
  // (X, dWh) run together and the second column tile reads it from L2; dW: (m, n, split) grid
  const int64_t mtile = MODE == DW ? (int64_t)blockIdx.x : (int64_t)blockIdx.x / g.ntiles;
  const int ntile = MODE == DW ? (int)blockIdx.y : (int)(blockIdx.x % g.ntiles);
  const int64_t m0 = mtile * BM;
  const int n0 = ntile * BN;
  const int64_t kb0 = (int64_t)blockIdx.z * g.kb_split;
  const int64_t kb1 = g.kb_total < kb0 + g.kb_split ? g.kb_total : kb0 + g.kb_split;
  const int nkb = kb1 > kb0 ? (int)(kb1 - kb0) : 0;
  const uint32_t full0 = smem_u32(bars), empty0 = smem_u32(bars + STAGES), done = smem_u32(bars + 2 * STAGES);

  if (MODE == FWD) {
    for (int c = threadIdx.x; c < BN; c += THREADS) {
      const bool ok = n0 + c < g.Nc;
      s_al[c] = ok ? g.al[n0 + c] : 0.f;
      s_ar[c] = ok ? g.ar[n0 + c] : 0.f;
    }
  }
  if (warp == 0) {
    if (lane == 0) {
      prefetch_tmap(&tmA);
      prefetch_tmap(&tmB);
      if (MODE != DW) prefetch_tmap(&tmO);
      for (int s = 0; s < STAGES; ++s) {
        mbar_init(full0 + 8 * s, 1);
        mbar_init(empty0 + 8 * s, 1);
      }
      mbar_init(done, 1);
      asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    }
    __syncwarp();
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tslot)),
                 "r"((uint32_t)TL::TMEM_COLS)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tslot;

  if (warp == 0 && lane == 0) {
    // ---- TMA producer ----
    for (int i = 0; i < nkb; ++i) {
      const int s = i % STAGES;
      const uint32_t ph = (uint32_t)(i / STAGES) & 1u;
      mbar_wait(empty0 + 8 * s, ph ^ 1u);
      const uint32_t full = full0 + 8 * s;
      mbar_expect_tx(full, TL::STAGE);
      const uint32_t sa = smem_u32(smem + s * TL::STAGE), sb = sa + TL::A_BYTES;
      const int32_t k = (int32_t)((kb0 + i) * BK);
      if constexpr (A_MN) {          // dW: X[row = k][k_in = m], two 64-wide m boxes
        tma_load_2d(sa, &tmA, (int32_t)m0, k, full);
        tma_load_2d(sa + 8192, &tmA, (int32_t)m0 + 64, k, full);
      } else {                        // K-major A: one 128-row box of 64 K
        tma_load_2d(sa, &tmA, k, (int32_t)m0, full);
      }
      if constexpr (B_MN) {          // B[k][n]: BN/64 boxes of 64 k-rows x 64 n
#pragma unroll
        for (int j = 0; j < BN / 64; ++j) tma_load_2d(sb + j * 8192, &tmB, n0 + 64 * j, k, full);
      } else {                        // K-major B: one BN-row box of 64 K
        tma_load_2d(sb, &tmB, k, n0, full);
      }
    }
  } else if (warp == 1 && lane == 0) {
    // ---- MMA issuer (one thread) ----
    constexpr uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((A_MN ? 1u : 0u) << 15) |
                               ((B_MN ? 1u : 0u) << 16) | ((uint32_t)(BN >> 3) << 17) | ((uint32_t)(BM >> 4) << 24);
    for (int i = 0; i < nkb; ++i) {
      const int s = i % STAGES;
      const uint32_t ph = (uint32_t)(i / STAGES) & 1u;
      mbar_wait(full0 + 8 * s, ph);
      tc_fence_after();
      const uint32_t sa = smem_u32(smem + s * TL::STAGE), sb = sa + TL::A_BYTES;
#pragma unroll
      for (int kk = 0; kk < BK / 16; ++kk) {
        const uint64_t da = A_MN ? sdesc(sa + kk * 2048, 8192, 1024) : sdesc(sa + kk * 32, 16, 1024);
        const uint64_t db = B_MN ? sdesc(sb + kk * 2048, 8192, 1024) : sdesc(sb + kk * 32, 16, 1024);
        umma_f16(tmem, da, db, idesc, (i | kk) ? 1u : 0u);
      }
      umma_commit(empty0 + 8 * s);   // frees the slot once these MMAs have read it
    }
    umma_commit(done);                // accumulator complete
  }
  __syncwarp();

  // ---- epilogue: TMEM -> registers -> global ----
  if (nkb > 0) mbar_wait(done, 0);
  tc_fence_after();
  const int row = warp * 32 + lane;
  const int64_t grow = m0 + row;
  const uint32_t taddr = tmem + ((uint32_t)(warp * 32) << 16);
  if constexpr (MODE == DW) {
    float *dst = static_cast<float *>(g.out) + ((int64_t)blockIdx.z * g.mpad + grow) * g.Nc + n0;
#pragma unroll 1
    for (int c0 = 0; c0 < BN; c0 += 32) {
      uint32_t r[32];
      if (nkb > 0) tmem_ld32(taddr + c0, r);
      else
#pragma unroll
        for (int q = 0; q < 32; ++q) r[q] = 0u;
      if (grow < g.M) {   // slab mode: M = mpad (every row); direct mode: M = in_dim rows of grad_w
#pragma unroll
        for (int q = 0; q < 8; ++q)
          *reinterpret_cast<uint4 *>(dst + c0 + 4 * q) = make_uint4(r[4 * q], r[4 * q + 1], r[4 * q + 2], r[4 * q + 3]);
      }
    }
  } else {
    // bf16 tile -> shared memory (the operand ring is free once the accumulator is complete),
    // laid out as BN/64 TMA boxes of [128 rows][128 B] with the 128-byte swizzle (conflict-free
    // row-per-thread writes), then TMA bulk stores (rows past M / columns past Nc are clipped)
    const bool live = grow < g.M;
    const uint32_t obase = smem_u32(smem);
    float el_acc = 0.f, er_acc = 0.f;
#pragma unroll 1
    for (int c0 = 0; c0 < BN; c0 += 32) {
      uint32_t r[32];
      tmem_ld32(taddr + c0, r);
      uint32_t p[16];
#pragma unroll
      for (int q = 0; q < 16; ++q) p[q] = bf2(__uint_as_float(r[2 * q]), __uint_as_float(r[2 * q + 1]));
      const uint32_t box = obase + (uint32_t)(c0 / 64) * (BM * 128) + (uint32_t)row * 128;
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const uint32_t u = (uint32_t)((c0 % 64) / 8 + q);
        asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(box + ((u ^ (uint32_t)(row & 7)) << 4)),
                     "r"(p[4 * q]), "r"(p[4 * q + 1]), "r"(p[4 * q + 2]), "r"(p[4 * q + 3])
                     : "memory");
      }
      if constexpr (MODE == FWD) {
        // el/er from the STORED (bf16-rounded) Wh, head by head (FH values per head segment)
#pragma unroll
        for (int sgm = 0; sgm < 32 / FH; ++sgm) {
#pragma unroll
          for (int q = 0; q < FH; q += 2) {
            const uint32_t w2 = p[(sgm * FH + q) / 2];
            const float x0 = __uint_as_float(w2 << 16), x1 = __uint_as_float(w2 & 0xffff0000u);
            const int c = c0 + sgm * FH + q;
            el_acc = fmaf(s_al[c], x0, el_acc);
            el_acc = fmaf(s_al[c + 1], x1, el_acc);
            er_acc = fmaf(s_ar[c], x0, er_acc);
            er_acc = fmaf(s_ar[c + 1], x1, er_acc);
          }
          const int cend = c0 + (sgm + 1) * FH;       // columns of this tile consumed so far
          if (cend % g.F == 0) {                       // a head is complete
            const int h = (n0 + cend) / g.F - 1;
            if (live && n0 + cend <= g.Nc) {
              g.el[(g.ctx_row0 + grow) * g.H + h] = el_acc;
              g.er[(g.ctx_row0 + grow) * g.H + h] = er_acc;
            }
            el_acc = 0.f;
            er_acc = 0.f;
          }
        }
      }
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // st.shared -> visible to the TMA engine
    __syncthreads();
    if (threadIdx.x == 0) {
#pragma unroll
      for (int j = 0; j < BN / 64; ++j)
        if (n0 + 64 * j < g.Nc) tma_store_2d(&tmO, obase + (uint32_t)j * (BM * 128), n0 + 64 * j, (int32_t)m0);
      asm volatile("cp.async.bulk.commit_group;" ::: "memory");
      asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");   // smem may be released after this
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 0) {
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"((uint32_t)TL::TMEM_COLS)
                 : "memory");
  }
}


// ---------------- persistent, warp-specialised form (fwd and dX) ----------------
// One CTA per SM loops over output tiles (tile t: row tile t / ntiles, column tile t % ntiles, so
// consecutive tiles share their A rows through L2).  Warp 0 (one lane) streams A/B k-blocks through
// a STAGES-deep TMA ring across tile boundaries; warp 1 (one lane) issues tcgen05.mma into one of
// TWO TMEM accumulators; warps 2-5 drain the other accumulator at the same time: tcgen05.ld ->
// bf16 -> swizzled shared-memory box -> TMA store (two 64-column boxes in flight), el/er on the way.
// So loads, MMAs and the epilogue of consecutive tiles overlap; barriers: full/empty per ring slot,
// tmem_full/tmem_empty per accumulator.
// EPI epilogue warpgroups (1 or 2): warpgroup e drains columns [e BN/EPI, (e+1) BN/EPI) of the
// accumulator (TMEM lanes are tied to warp % 4, so two warpgroups split the columns, not the rows).
template <int BN, int EPI> struct PTiles {
  static constexpr int A_BYTES = BM * BK * 2, B_BYTES = BN * BK * 2, STAGE = A_BYTES + B_BYTES;
  static constexpr int OUT_BOX = BM * 128;                      // one 64-column bf16 box, 16 KB
  static constexpr int OUT = 2 * EPI * OUT_BOX;                 // two boxes in flight per warpgroup
  static constexpr int STAGES = (216 * 1024 - OUT) / STAGE > 8 ? 8 : (216 * 1024 - OUT) / STAGE;
  static constexpr int ACC_COLS = BN <= 32 ? 32 : BN <= 64 ? 64 : BN <= 128 ? 128 : 256;
  static constexpr int TMEM_COLS = 2 * ACC_COLS;
  static constexpr size_t SMEM = 1024 + (size_t)STAGES * STAGE + OUT + 512;   // + 8 KB static (a_l, a_r)
  static constexpr int THREADS = 64 + 128 * EPI;
};

template <int MODE, int BN, int FH, int EPI>
__global__ void __launch_bounds__(PTiles<BN, EPI>::THREADS, 1)
    umma_gemm_persistent(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                         const __grid_constant__ CUtensorMap tmO, const Args g) {
  using TL = PTiles<BN, EPI>;
  constexpr int PTHREADS = TL::THREADS, CW = BN / EPI;    // columns per epilogue warpgroup
  static_assert(CW % 64 == 0 || EPI == 1, "a warpgroup's columns are whole 64-column boxes");
  constexpr int STAGES = TL::STAGES;
  static_assert(MODE == FWD || MODE == DX, "persistent kernel: fwd and dX");
  constexpr bool B_MN = MODE == FWD;
  extern __shared__ uint8_t smem_raw[];
  uint8_t *smem = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~(uintptr_t)1023);
  uint8_t *outb = smem + STAGES * TL::STAGE;                         // 2 output boxes per warpgroup
  uint64_t *bars = reinterpret_cast<uint64_t *>(outb + TL::OUT);
  // bars: full[S], empty[S], tfull[2], tempty[2]
  uint32_t *tslot = reinterpret_cast<uint32_t *>(bars + 2 * STAGES + 4);
  __shared__ __align__(16) float s_alr[2][1024];   // a_l, a_r (static: the compiler knows they are shared)
  float *s_al = s_alr[0], *s_ar = s_alr[1];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t full0 = smem_u32(bars), empty0 = smem_u32(bars + STAGES);
  const uint32_t tfull0 = smem_u32(bars + 2 * STAGES), tempty0 = smem_u32(bars + 2 * STAGES + 2);
  const int64_t mtiles = (g.M + BM - 1) / BM, ntile_total = mtiles * g.ntiles;
  const int nkb = (int)g.kb_total;

  if (MODE == FWD)
    for (int c = threadIdx.x; c < g.Nc; c += PTHREADS) { s_al[c] = g.al[c]; s_ar[c] = g.ar[c]; }
  if (warp == 0 && lane == 0) {
    prefetch_tmap(&tmA);
    prefetch_tmap(&tmB);
    prefetch_tmap(&tmO);
    for (int s2 = 0; s2 < STAGES; ++s2) {
      mbar_init(full0 + 8 * s2, 1);
      mbar_init(empty0 + 8 * s2, 1);
    }
    for (int a2 = 0; a2 < 2; ++a2) {
      mbar_init(tfull0 + 8 * a2, 1);
      mbar_init(tempty0 + 8 * a2, 4 * EPI);       // one arrive per epilogue warp
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tslot)),
                 "r"((uint32_t)TL::TMEM_COLS)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tslot;

  if (warp == 0) {
    if (lane == 0) {   // ---- TMA producer: k-blocks of every tile of this CTA, through the ring ----
      // The A operand (X / dWh rows) streams from HBM: its k-blocks are also prefetched into L2
      // PF k-blocks ahead (across tile boundaries), so a ring slot waits on an L2 hit, not on DRAM
      // latency (the ring is only STAGES deep; B is small and L2-resident anyway).
      constexpr int PF = 6;
      int64_t pt = blockIdx.x;
      int pi = 0;
      for (int q = 0; q < PF; ++q) {   // warm-up: the first PF k-blocks
        if (pt < ntile_total) tma_prefetch_2d(&tmA, pi * BK, (int32_t)((pt / g.ntiles) * BM));
        if (++pi == nkb) { pi = 0; pt += gridDim.x; }
      }
      int64_t kc = 0;
      for (int64_t t = blockIdx.x; t < ntile_total; t += gridDim.x) {
        const int32_t m0 = (int32_t)((t / g.ntiles) * BM), n0 = (int32_t)((t % g.ntiles) * BN);
        for (int i = 0; i < nkb; ++i, ++kc) {
          if (pt < ntile_total) tma_prefetch_2d(&tmA, pi * BK, (int32_t)((pt / g.ntiles) * BM));
          if (++pi == nkb) { pi = 0; pt += gridDim.x; }
          const int s2 = (int)(kc % STAGES);
          mbar_wait(empty0 + 8 * s2, (uint32_t)((kc / STAGES) & 1) ^ 1u);
          const uint32_t full = full0 + 8 * s2;
          mbar_expect_tx(full, TL::STAGE);
          const uint32_t sa = smem_u32(smem + s2 * TL::STAGE), sb = sa + TL::A_BYTES;
          const int32_t k = i * BK;
          tma_load_2d(sa, &tmA, k, m0, full);
          if constexpr (B_MN) {
#pragma unroll
            for (int j = 0; j < BN / 64; ++j) tma_load_2d(sb + j * 8192, &tmB, n0 + 64 * j, k, full);
          } else {
            tma_load_2d(sb, &tmB, k, n0, full);
          }
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {   // ---- MMA issuer ----
      constexpr uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((B_MN ? 1u : 0u) << 16) |
                                 ((uint32_t)(BN >> 3) << 17) | ((uint32_t)(BM >> 4) << 24);
      int64_t kc = 0, it = 0;
      for (int64_t t = blockIdx.x; t < ntile_total; t += gridDim.x, ++it) {
        const int acc = (int)(it & 1);
        mbar_wait(tempty0 + 8 * acc, (uint32_t)((it >> 1) & 1) ^ 1u);   // the epilogue drained it
        tc_fence_after();
        const uint32_t td = tmem + (uint32_t)(acc * TL::ACC_COLS);
        for (int i = 0; i < nkb; ++i, ++kc) {
          const int s2 = (int)(kc % STAGES);
          mbar_wait(full0 + 8 * s2, (uint32_t)((kc / STAGES) & 1));
          tc_fence_after();
          const uint32_t sa = smem_u32(smem + s2 * TL::STAGE), sb = sa + TL::A_BYTES;
#pragma unroll
          for (int kk = 0; kk < BK / 16; ++kk) {
            const uint64_t da = sdesc(sa + kk * 32, 16, 1024);
            const uint64_t db = B_MN ? sdesc(sb + kk * 2048, 8192, 1024) : sdesc(sb + kk * 32, 16, 1024);
            umma_f16(td, da, db, idesc, (i | kk) ? 1u : 0u);
          }
          umma_commit(empty0 + 8 * s2);
        }
        umma_commit(tfull0 + 8 * acc);
      }
    }
  } else {
    // ---- epilogue warps 2..: TMEM lanes 32 (warp % 4) .. +31 = tile rows; warpgroup ewg takes
    // columns [ewg CW, (ewg+1) CW) of each tile ----
    const int ew = warp & 3, ewg = (warp - 2) / 4, row = ew * 32 + lane, et = threadIdx.x - 64 - 128 * ewg;
    const uint32_t obase = smem_u32(outb) + (uint32_t)(ewg * 2 * TL::OUT_BOX);
    const int bar_id = 1 + ewg;
    int64_t it = 0, chunk = 0;
    for (int64_t t = blockIdx.x; t < ntile_total; t += gridDim.x, ++it) {
      const int64_t m0 = (t / g.ntiles) * BM;
      const int n0 = (int)((t % g.ntiles) * BN);
      const int acc = (int)(it & 1);
      mbar_wait(tfull0 + 8 * acc, (uint32_t)((it >> 1) & 1));
      tc_fence_after();
      const uint32_t taddr = tmem + (uint32_t)(acc * TL::ACC_COLS) + ((uint32_t)(ew * 32) << 16);
      const int64_t grow = m0 + row;
      const bool live = grow < g.M;
      float el0 = 0.f, el1 = 0.f, er0 = 0.f, er1 = 0.f;   // even / odd column partial sums (FFMA2)
#pragma unroll 1
      for (int c64 = ewg * CW; c64 < (ewg + 1) * CW; c64 += 64, ++chunk) {
        const int b = (int)(chunk & 1);
        // the TMA store that last read box b must be done before it is rewritten
        if (et == 0) asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
        asm volatile("bar.sync %0, 128;" ::"r"(bar_id) : "memory");
        const uint32_t box = obase + (uint32_t)b * TL::OUT_BOX + (uint32_t)row * 128;
#pragma unroll
        for (int h32 = 0; h32 < 2; ++h32) {
          const int c0 = c64 + 32 * h32;
          uint32_t r[32];
          tmem_ld32(taddr + c0, r);
          uint32_t p[16];
#pragma unroll
          for (int q = 0; q < 16; ++q) p[q] = bf2(__uint_as_float(r[2 * q]), __uint_as_float(r[2 * q + 1]));
#pragma unroll
          for (int q = 0; q < 4; ++q) {
            const uint32_t u = (uint32_t)(4 * h32 + q);
            asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(box + ((u ^ (uint32_t)(row & 7)) << 4)),
                         "r"(p[4 * q]), "r"(p[4 * q + 1]), "r"(p[4 * q + 2]), "r"(p[4 * q + 3])
                         : "memory");
          }
          if constexpr (MODE == FWD) {   // el/er from the stored (bf16-rounded) Wh, head by head
#pragma unroll
            for (int sgm = 0; sgm < 32 / FH; ++sgm) {
#pragma unroll
              for (int q = 0; q < FH; q += 4) {   // 4 columns: one 16-byte broadcast load of a_l and a_r each
                const uint32_t wa = p[(sgm * FH + q) / 2], wb = p[(sgm * FH + q) / 2 + 1];
                const float x0 = __uint_as_float(wa << 16), x1 = __uint_as_float(wa & 0xffff0000u);
                const float x2 = __uint_as_float(wb << 16), x3 = __uint_as_float(wb & 0xffff0000u);
                const int c = n0 + c0 + sgm * FH + q;
                const float4 al4 = *reinterpret_cast<const float4 *>(s_al + c);
                const float4 ar4 = *reinterpret_cast<const float4 *>(s_ar + c);
                ffma2(el0, el1, x0, x1, al4.x, al4.y);
                ffma2(el0, el1, x2, x3, al4.z, al4.w);
                ffma2(er0, er1, x0, x1, ar4.x, ar4.y);
                ffma2(er0, er1, x2, x3, ar4.z, ar4.w);
              }
              const int cend = c0 + (sgm + 1) * FH;
              if (cend % g.F == 0) {
                const int h = (n0 + cend) / g.F - 1;
                if (live) {
                  g.el[(g.ctx_row0 + grow) * g.H + h] = el0 + el1;
                  g.er[(g.ctx_row0 + grow) * g.H + h] = er0 + er1;
                }
                el0 = el1 = er0 = er1 = 0.f;
              }
            }
          }
        }
        if (c64 + 64 >= (ewg + 1) * CW) {   // this thread's TMEM reads of the tile are done: release
          tc_fence_before();
          __syncwarp();
          if (lane == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(tempty0 + 8 * acc) : "memory");
        }
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        asm volatile("bar.sync %0, 128;" ::"r"(bar_id) : "memory");
        if (et == 0) {
          if (n0 + c64 < g.Nc) tma_store_2d(&tmO, obase + (uint32_t)b * TL::OUT_BOX, n0 + c64, (int32_t)m0);
          asm volatile("cp.async.bulk.commit_group;" ::: "memory");
        }
      }
    }
    if (et == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
  }
  __syncwarp();
  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"((uint32_t)TL::TMEM_COLS)
                 : "memory");
  }
}

// dW: fixed-order sum of the split partials (deterministic), fp32
__global__ void __launch_bounds__(256) dw_reduce_kernel(const float *parts, int splits, int64_t mpad, int K, int D,
                                                        float *out) {
  const int64_t n4 = (int64_t)K * D / 4;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n4; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t e = 4 * i;
    const int64_t k = e / D, d = e % D;
    float4 s = make_float4(0.f, 0.f, 0.f, 0.f);
    int z = 0;
    for (; z + 8 <= splits; z += 8) {   // 8 independent loads in flight, then the fixed-order adds
      float4 v[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) v[u] = *reinterpret_cast<const float4 *>(parts + ((int64_t)(z + u) * mpad + k) * D + d);
#pragma unroll
      for (int u = 0; u < 8; ++u) { s.x += v[u].x; s.y += v[u].y; s.z += v[u].z; s.w += v[u].w; }
    }
    for (; z < splits; ++z) {
      const float4 v = *reinterpret_cast<const float4 *>(parts + ((int64_t)z * mpad + k) * D + d);
      s.x += v.x; s.y += v.y; s.z += v.z; s.w += v.w;
    }
    *reinterpret_cast<float4 *>(out + e) = s;
  }
}

// ------------------------------------------------------------------ host side
PFN_cuTensorMapEncodeTiled_v12000 encoder() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    void *p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
  });
  return fn;
}

// 2-D bf16 tensor map: `inner` contiguous elements per row, `outer` rows `ld` elements apart,
// box {box_inner (<= 64: 128 B), box_outer}, 128-byte swizzle, zero fill out of bounds
mega_status tmap_2d(CUtensorMap *m, const void *base, uint64_t inner, uint64_t outer, int64_t ld, uint32_t box_inner,
                    uint32_t box_outer) {
  auto enc = encoder();
  if (!enc) return fail(MEGA_ERR_CUDA, "cuTensorMapEncodeTiled unavailable (driver entry point)");
  const cuuint64_t dims[2] = {inner, outer};
  const cuuint64_t strides[1] = {(cuuint64_t)ld * 2};
  const cuuint32_t box[2] = {box_inner, box_outer};
  const cuuint32_t es[2] = {1, 1};
  CUresult r = enc(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void *>(base), dims, strides, box, es,
                   CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return fail(MEGA_ERR_CUDA, "cuTensorMapEncodeTiled failed (" + std::to_string((int)r) + ")");
  return MEGA_OK;
}

int sm_count() {
  static int sms = 0;
  if (!sms) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    if (sms <= 0) sms = 148;
  }
  return sms;
}

template <int MODE, int BN, int FH>
mega_status launch(const CUtensorMap &a, const CUtensorMap &b, const CUtensorMap &o, const Args &g, dim3 grid,
                   cudaStream_t st) {
  auto k = umma_gemm_kernel<MODE, BN, FH>;
  const size_t smem = Tiles<BN>::SMEM;
  static bool attr = false;  // per instantiation
  if (!attr) {
    cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return fail(MEGA_ERR_CUDA, std::string("umma smem attribute: ") + cudaGetErrorString(e));
    attr = true;
  }
  k<<<grid, THREADS, smem, st>>>(a, b, o, g);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return fail(MEGA_ERR_CUDA, std::string("umma_gemm_kernel: ") + cudaGetErrorString(e));
  return MEGA_OK;
}

template <int MODE, int BN, int FH, int EPI>
mega_status launch_persistent_e(const CUtensorMap &a, const CUtensorMap &b, const CUtensorMap &o, const Args &g,
                                cudaStream_t st) {
  auto k = umma_gemm_persistent<MODE, BN, FH, EPI>;
  const size_t smem = PTiles<BN, EPI>::SMEM;
  static bool attr = false;  // per instantiation
  if (!attr) {
    cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return fail(MEGA_ERR_CUDA, std::string("umma smem attribute: ") + cudaGetErrorString(e));
    attr = true;
  }
  const int64_t tiles = ((g.M + BM - 1) / BM) * g.ntiles;
  const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(tiles, sm_count()));
  k<<<grid, PTiles<BN, EPI>::THREADS, smem, st>>>(a, b, o, g);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return fail(MEGA_ERR_CUDA, std::string("umma_gemm_persistent: ") + cudaGetErrorString(e));
  return MEGA_OK;
}
// two epilogue warpgroups when each half of the tile is whole 64-column boxes holding whole heads
template <int MODE, int BN, int FH>
mega_status launch_persistent(const CUtensorMap &a, const CUtensorMap &b, const CUtensorMap &o, const Args &g,
                              cudaStream_t st) {
  if constexpr (BN % 128 == 0) {
    if (MODE == DX || (BN / 2) % g.F == 0) return launch_persistent_e<MODE, BN, FH, 2>(a, b, o, g, st);
  }
  return launch_persistent_e<MODE, BN, FH, 1>(a, b, o, g, st);
}

}  // namespace umma

using namespace umma;

// Wh = X W (+ el/er of each head into the ctx planes).  bf16.  D <= 256 per tile:
// BN = min(D, 256) must be a multiple of head_dim (so a tile holds whole heads) and of 64.
mega_status umma_project_fwd(const void *x, int64_t ldx, int64_t rows, int in_dim, const void *w, int heads,
                             int head_dim, const float *al, const float *ar, void *feat, int64_t ldf, float *el,
                             float *er, int64_t ctx_row0, cudaStream_t st) {
  const int D = heads * head_dim;
  const int BN = std::min(D, 256);
  if (D % 64 || BN % head_dim || head_dim % 8)
    return fail(MEGA_ERR_UNSUPPORTED, "tcgen05 projection: D must be a multiple of 64 and head_dim divide min(D, 256)");
  CUtensorMap ta, tb, to;
  mega_status rc;
  if ((rc = tmap_2d(&ta, x, (uint64_t)in_dim, (uint64_t)rows, ldx, 64, BM)) != MEGA_OK) return rc;
  if ((rc = tmap_2d(&tb, w, (uint64_t)D, (uint64_t)in_dim, D, 64, 64)) != MEGA_OK) return rc;
  if ((rc = tmap_2d(&to, feat, (uint64_t)D, (uint64_t)rows, ldf, 64, BM)) != MEGA_OK) return rc;
  Args g{};
  g.M = rows; g.Nc = D; g.kb_total = (in_dim + BK - 1) / BK; g.kb_split = g.kb_total;
  g.out = feat; g.ldo = ldf; g.el = el; g.er = er; g.al = al; g.ar = ar; g.H = heads; g.F = head_dim;
  g.ctx_row0 = ctx_row0;
  g.ntiles = D / BN;
  const dim3 grid((unsigned)(((rows + BM - 1) / BM) * g.ntiles), 1, 1);
  const int fh = std::min(head_dim, 32);
  if (BN == 256) {
    if (fh == 32) return launch_persistent<FWD, 256, 32>(ta, tb, to, g, st);
    if (fh == 16) return launch_persistent<FWD, 256, 16>(ta, tb, to, g, st);
    return launch_persistent<FWD, 256, 8>(ta, tb, to, g, st);
  }
  if (BN == 128) {
    if (fh == 32) return launch_persistent<FWD, 128, 32>(ta, tb, to, g, st);
    if (fh == 16) return launch_persistent<FWD, 128, 16>(ta, tb, to, g, st);
    return launch_persistent<FWD, 128, 8>(ta, tb, to, g, st);
  }
  if (BN == 192) {
    if (fh == 32) return launch_persistent<FWD, 192, 32>(ta, tb, to, g, st);
    if (fh == 16) return launch_persistent<FWD, 192, 16>(ta, tb, to, g, st);
    return launch_persistent<FWD, 192, 8>(ta, tb, to, g, st);
  }
  if (fh == 32) return launch_persistent<FWD, 64, 32>(ta, tb, to, g, st);
  if (fh == 16) return launch_persistent<FWD, 64, 16>(ta, tb, to, g, st);
  return launch_persistent<FWD, 64, 8>(ta, tb, to, g, st);
}

// dX[rows][in_dim] = dWh W^T (bf16 out).  K = D (multiple of 64).  Columns are written in
// 8-wide (16-byte) vectors up to round_up(in_dim, 8) (<= ldgx): the ones past in_dim get 0
// (W rows past in_dim read as zeros), i.e. the zero padding of a padded X.
mega_status umma_project_dx(const void *gf, int64_t ldgf, int64_t rows, int in_dim, const void *w, int D, void *gx,
                            int64_t ldgx, cudaStream_t st) {
  if (D % 64) return fail(MEGA_ERR_UNSUPPORTED, "tcgen05 dX: D % 64 required");
  const int BN = in_dim >= 256 ? 256 : (in_dim >= 128 ? 128 : 64);
  CUtensorMap ta, tb, to;
  mega_status rc;
  if ((rc = tmap_2d(&ta, gf, (uint64_t)D, (uint64_t)rows, ldgf, 64, BM)) != MEGA_OK) return rc;
  if ((rc = tmap_2d(&tb, w, (uint64_t)D, (uint64_t)in_dim, D, 64, BN)) != MEGA_OK) return rc;
  if ((rc = tmap_2d(&to, gx, (uint64_t)((in_dim + 7) / 8 * 8), (uint64_t)rows, ldgx, 64, BM)) != MEGA_OK) return rc;
  Args g{};
  g.M = rows; g.Nc = (in_dim + 7) / 8 * 8; g.kb_total = D / BK; g.kb_split = g.kb_total; g.out = gx; g.ldo = ldgx;
  g.ntiles = (in_dim + BN - 1) / BN;
  const dim3 grid((unsigned)(((rows + BM - 1) / BM) * g.ntiles), 1, 1);
  if (BN == 256) return launch_persistent<DX, 256, 32>(ta, tb, to, g, st);
  if (BN == 128) return launch_persistent<DX, 128, 32>(ta, tb, to, g, st);
  return launch_persistent<DX, 64, 32>(ta, tb, to, g, st);
}

// dW reductions of at most kUnsplitKb 64-row K blocks run in one CTA per output tile, writing grad_w
// directly (no partials, no reduction launch).  MEGA_DW_UNSPLIT_KB: 8 (default) / 32 / 128 measured
// 0.160 / 0.167 / 0.167 ms per zinc-b64 step and 0.206 / 0.210 / 0.289 for zinc-b256 (profiles/r02/dw_split/)
int unsplit_kb() {
  static int v = -1;
  if (v < 0) {
    const char *e = std::getenv("MEGA_DW_UNSPLIT_KB");
    v = e ? std::atoi(e) : 8;
  }
  return v;
}
// workspace of umma_project_dw: split partials
void umma_dw_plan(int64_t rows, int in_dim, int D, int &splits, int64_t &mpad, size_t &bytes) {
  const int kUnsplitKb = unsplit_kb();
  const int BN = std::min(D, 256);
  const int64_t mt = (in_dim + BM - 1) / BM, nt = (D + BN - 1) / BN;
  const int64_t kbt = (rows + BK - 1) / BK;
  int64_t s = (2 * (int64_t)sm_count() + mt * nt - 1) / (mt * nt);
  s = std::max<int64_t>(1, std::min<int64_t>(s, kbt));
  // very short reductions (<= 512 rows) run unsplit, writing grad_w directly (one launch); longer
  // ones split: one CTA walking ~100 K blocks was measured slower (zinc-b256 step 0.26 -> 0.31 ms)
  // than a split GEMM plus its reduction
  if (kbt <= kUnsplitKb) s = 1;
  const int64_t per = std::max<int64_t>(kbt <= kUnsplitKb ? kbt : 4, (kbt + s - 1) / s);   // >= 4 K blocks per split
  splits = (int)((kbt + per - 1) / per);   // every split non-empty
  mpad = mt * BM;
  bytes = splits == 1 ? 256 : (size_t)splits * (size_t)mpad * (size_t)D * 4;
}

// dW[in_dim][D] = X^T dWh (fp32 out), split over rows, fixed-order reduce.
mega_status umma_project_dw(const void *x, int64_t ldx, const void *gf, int64_t ldgf, int64_t rows, int in_dim, int D,
                            float *gw, void *ws, size_t ws_bytes, cudaStream_t st) {
  if (D % 64) return fail(MEGA_ERR_UNSUPPORTED, "tcgen05 dW: D % 64 required");
  int splits;
  int64_t mpad;
  size_t need;
  umma_dw_plan(rows, in_dim, D, splits, mpad, need);
  if (ws_bytes < need) return fail(MEGA_ERR_OUT_OF_MEMORY, "projection workspace too small (mega_project_workspace_bytes)");
  const int BN = std::min(D, 256);
  CUtensorMap ta, tb;
  mega_status rc;
  if ((rc = tmap_2d(&ta, x, (uint64_t)in_dim, (uint64_t)rows, ldx, 64, 64)) != MEGA_OK) return rc;
  if ((rc = tmap_2d(&tb, gf, (uint64_t)D, (uint64_t)rows, ldgf, 64, 64)) != MEGA_OK) return rc;
  Args g{};
  g.M = mpad; g.Nc = D; g.kb_total = (rows + BK - 1) / BK; g.kb_split = (g.kb_total + splits - 1) / splits;
  g.out = ws; g.mpad = mpad;
  if (splits == 1) {   // direct: the one partial is grad_w itself (rows < in_dim written)
    g.M = in_dim;
    g.out = gw;
    g.mpad = 0;
  }
  const dim3 grid((unsigned)(mpad / BM), (unsigned)(D / BN), (unsigned)splits);
  if (BN == 256) rc = launch<DW, 256, 32>(ta, tb, ta, g, grid, st);
  else if (BN == 128) rc = launch<DW, 128, 32>(ta, tb, ta, g, grid, st);
  else if (BN == 192) rc = launch<DW, 192, 32>(ta, tb, ta, g, grid, st);
  else rc = launch<DW, 64, 32>(ta, tb, ta, g, grid, st);
  if (rc != MEGA_OK || splits == 1) return rc;
  const int64_t n4 = (int64_t)in_dim * D / 4;
  const int blocks = (int)std::min<int64_t>((n4 + 255) / 256, 4 * sm_count());
  dw_reduce_kernel<<<std::max(blocks, 1), 256, 0, st>>>(static_cast<const float *>(ws), splits, mpad, in_dim, D, gw);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return fail(MEGA_ERR_CUDA, std::string("dw_reduce_kernel: ") + cudaGetErrorString(e));
  return MEGA_OK;
}

}  // namespace mega
