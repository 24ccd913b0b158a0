// Measurement helper (SURVEY §8(d)-d2 calibration, not on the hot path): the
// achievable bandwidth of gathering rows of a table by an index list, the
// access pattern of the attention kernels.  Each warp sums the rows named by
// 32 consecutive indices (U rows in flight per lane) and writes one partial
// per warp, so nothing is optimised away.
#include <cuda_runtime.h>

#include <cstdlib>

#include "mega_internal.h"
#include "kern_common.cuh"

namespace mega {
namespace {
using namespace kern;

template <int V, int U>
__global__ void __launch_bounds__(256) gather_kernel(const uint4 *table, int64_t row_vecs, const int32_t *idx,
                                                     int64_t n, float *sink, int pol_mode) {
  const uint64_t pol = pol_mode == 1 ? policy_first() : (pol_mode == 2 ? policy_last() : policy_normal());
  const int lane = threadIdx.x & 31;
  const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  uint32_t acc = 0;
  for (int64_t b = warp * 32; b < n; b += nwarps * 32) {
    const int my = b + lane < n ? __ldg(idx + b + lane) : -1;
    const int cnt = (n - b) < 32 ? (int)(n - b) : 32;
    for (int k0 = 0; k0 < cnt; k0 += U) {
      uint4 r[U][V];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const int j = __shfl_sync(0xffffffffu, my, (k0 + u) & 31);
        if (k0 + u < cnt) {
#pragma unroll
          for (int v = 0; v < V; ++v) r[u][v] = ldg16_pol(table + (int64_t)j * row_vecs + v * 32 + lane, pol);
        } else {
#pragma unroll
          for (int v = 0; v < V; ++v) r[u][v] = make_uint4(0, 0, 0, 0);
        }
      }
#pragma unroll
      for (int u = 0; u < U; ++u)
#pragma unroll
        for (int v = 0; v < V; ++v) acc ^= r[u][v].x ^ r[u][v].y ^ r[u][v].z ^ r[u][v].w;
    }
  }
  if (lane == 0) sink[warp] = (float)acc;
}

}  // namespace
}  // namespace mega

extern "C" mega_status mega_calib_gather(const void *table, int64_t rows, int row_bytes, const int32_t *idx,
                                         int64_t n, float *sink, int64_t sink_len, mega_stream_t stream) {
  using namespace mega;
  clear_error();
  if (!table || !idx || !sink || rows <= 0 || n < 0) return fail(MEGA_ERR_INVALID_ARGUMENT, "bad arguments");
  int dev = 0, sms = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  // analysis knobs: MEGA_CALIB_BPS blocks per SM (default 8), MEGA_CALIB_POL L2 policy (0 normal, 1 first, 2 last)
  const char *e_bps = getenv("MEGA_CALIB_BPS"), *e_pol = getenv("MEGA_CALIB_POL");
  const int bps = e_bps ? atoi(e_bps) : 8, pm = e_pol ? atoi(e_pol) : 0;
  if (bps < 1 || bps > 8) return fail(MEGA_ERR_INVALID_ARGUMENT, "MEGA_CALIB_BPS must be 1..8");
  const int blocks = sms * bps;
  if (sink_len < (int64_t)blocks * 8) return fail(MEGA_ERR_OUT_OF_MEMORY, "sink must hold 8 * 8 * SMs floats");
  cudaStream_t st = (cudaStream_t)stream;
  const uint4 *t = static_cast<const uint4 *>(table);
  switch (row_bytes) {
    case 512: gather_kernel<1, 8><<<blocks, 256, 0, st>>>(t, 32, idx, n, sink, pm); break;
    case 1024: gather_kernel<2, 4><<<blocks, 256, 0, st>>>(t, 64, idx, n, sink, pm); break;
    case 2048: gather_kernel<4, 2><<<blocks, 256, 0, st>>>(t, 128, idx, n, sink, pm); break;
    default: return fail(MEGA_ERR_UNSUPPORTED, "row_bytes must be 512, 1024 or 2048");
  }
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? MEGA_OK : fail(MEGA_ERR_CUDA, cudaGetErrorString(e));
}
