// ks_prep.cu -- source preparation (scope row a1).
//
// Paper: Alg.1 l.3 computes vec_alpha = [||alpha_0||^2 ... ||alpha_{M-1}||^2]
// for the norm identity Eq.3.  The paper does
// not say where or how.  Here it runs once per ks_set_sources, on the device:
//   1. mu = mean of the sources (FP64 accumulation, fixed order) -- centring
//      is exact for the Gaussian (it depends on alpha - beta only) and shrinks
//      the cancellation of Eq.3 in FP32 (SS3, reading Q8/Q11);
//   2. per source: alpha_hat = alpha - mu (FP32), n = ||alpha_hat||^2 (FP64
//      accumulate), stored prescaled for the ex2-based exponent:
//      a = RN(2c * alpha_hat), na = RN(-c * n), c = log2(e)/(2h^2);
//      layout dimension-major so one TMA box brings a source tile's
//      coordinates, norms and weights into shared memory.
#include "ks_internal.h"

namespace ks {

// Each block sums a contiguous chunk of rows in a fixed order.  For K <= 256
// the 256 threads form rpp = 256/K row lanes x K dims (coalesced reads); the
// rpp lane sums of a dim are then added in lane order.  For K > 256 thread t
// owns dims t, t+256, ...
__global__ void source_mean_partial_kernel(const float* __restrict__ alpha, int64_t M, int K, int nparts,
                                           double* __restrict__ part) {
  __shared__ double red[256];
  const int b = blockIdx.x;
  const int t = threadIdx.x;
  const int64_t chunk = (M + nparts - 1) / nparts;
  const int64_t r0 = b * chunk;
  const int64_t r1 = (r0 + chunk < M) ? r0 + chunk : M;
  if (K <= 256) {
    const int rpp = 256 / K;
    const int ro = t / K, d = t % K;
    double s = 0.0;
    if (ro < rpp)
      for (int64_t r = r0 + ro; r < r1; r += rpp) s += (double)alpha[r * K + d];
    red[t] = s;
    __syncthreads();
    if (t < K) {
      double acc = 0.0;
      for (int q = 0; q < rpp; ++q) acc += red[q * K + t];
      part[(int64_t)b * K + t] = acc;
    }
  } else {
    for (int d = t; d < K; d += blockDim.x) {
      double s = 0.0;
      for (int64_t r = r0; r < r1; ++r) s += (double)alpha[r * K + d];
      part[(int64_t)b * K + d] = s;
    }
  }
}

// One warp per dimension: lanes sum the block partials in a fixed strided
// order, then a fixed shuffle tree (deterministic).
__global__ void source_mean_final_kernel(const double* __restrict__ part, int nparts, int64_t M, int K,
                                         int k_pad, float* __restrict__ mu) {
  const int d = (int)(((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5);
  const int lane = threadIdx.x & 31;
  if (d >= k_pad) return;
  double s = 0.0;
  if (d < K)
    for (int b = lane; b < nparts; b += 32) s += part[(int64_t)b * K + d];
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) s += __shfl_down_sync(0xffffffffu, s, o);
  if (lane == 0) mu[d] = (d < K && M > 0) ? (float)(s / (double)M) : 0.f;
}

cudaError_t launch_source_mean(const float* alpha, int64_t M, int K, int k_pad, double* part, int nparts,
                               float* mu, cudaStream_t st) {
  if (M > 0) {
    source_mean_partial_kernel<<<nparts, 256, 0, st>>>(alpha, M, K, nparts, part);
  }
  const int warps_per_block = 8;
  source_mean_final_kernel<<<(k_pad + warps_per_block - 1) / warps_per_block, 32 * warps_per_block, 0, st>>>(
      part, M > 0 ? nparts : 0, M, K, k_pad, mu);
  return cudaGetLastError();
}

// One thread per (padded) source column.
__global__ void prep_fp32_kernel(const float* __restrict__ alpha, const float* __restrict__ W, int64_t M,
                                 int64_t m_pad, int K, int k_pad, const float* __restrict__ mu, double c,
                                 float* __restrict__ src) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= m_pad) return;
  const bool live = i < M;
  const double c2 = 2.0 * c;
  double n = 0.0;
  for (int d = 0; d < k_pad; ++d) {
    float x = 0.f;
    if (live && d < K) x = alpha[i * K + d] - mu[d];  // FP32 centring, same op as the target side
    n += (double)x * (double)x;
    src[(int64_t)d * m_pad + i] = (float)(c2 * (double)x);
  }
  src[(int64_t)k_pad * m_pad + i] = live ? (float)(-c * n) : 0.f;
  src[(int64_t)(k_pad + 1) * m_pad + i] = live ? W[i] : 0.f;
}

cudaError_t launch_prep_fp32(const float* alpha, const float* W, int64_t M, int64_t m_pad, int K, int k_pad,
                             const float* mu, double c, float* src, cudaStream_t st) {
  if (m_pad == 0) return cudaSuccess;
  const int bs = 256;
  const int64_t nb = (m_pad + bs - 1) / bs;
  prep_fp32_kernel<<<(unsigned)nb, bs, 0, st>>>(alpha, W, M, m_pad, K, k_pad, mu, c, src);
  return cudaGetLastError();
}

}  // namespace ks
