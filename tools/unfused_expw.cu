// unfused_expw.cu -- the second pass of the fair unfused comparison design (NEXT-1, the
// paper's cuBLAS-Unfused, Alg.1): after cuBLAS SGEMM has written the
// target x source block G = (2c beta_hat) alpha_hat^T to HBM, ONE kernel reads every G_ji
// exactly once, adds the norms, clamps d^2 >= 0, exponentiates and multiplies by W:
//     V_jr = sum_i exp2(min(G_ji + na_i + nb_j, 0)) W_ir      (Alg.1 l.11-16 in one pass)
// so the unfused design moves 8 bytes per pair through HBM (GEMM write + this read), the
// least any design that materialises the block can.  A measurement baseline in tools/, not
// the product (libks.so's fused kernel never writes the block).
//
// Layout: G [n][M] row-major FP32 (one target row contiguous), na [M], nb [n], W [M][R],
// V [n][R].  One 256-thread block per target row: float4 loads along the row (coalesced),
// FP32 partials per thread, FP64 block reduction.  C ABI for ctypes (plain pointers).
#include <cuda_runtime.h>
#include <cstdint>

namespace {

constexpr int kThreads = 256;
constexpr int kMaxR = 16;

template <int RR>
__global__ void __launch_bounds__(kThreads) expw_rows_kernel(const float* __restrict__ G, const float* __restrict__ na,
                                                          const float* __restrict__ nb, const float* __restrict__ W,
                                                          float* __restrict__ V, int64_t M, int R) {
  const int64_t j = blockIdx.x;
  const float* g = G + j * M;
  const float nbj = nb[j];
  float acc[RR];
#pragma unroll
  for (int r = 0; r < RR; ++r) acc[r] = 0.f;
  const int64_t M4 = (M & 3) == 0 ? M : 0;  // float4 path when rows stay 16-byte aligned
  for (int64_t i = 4 * (int64_t)threadIdx.x; i < M4; i += 4 * kThreads) {
    const float4 x = __ldcs(reinterpret_cast<const float4*>(g + i));  // streamed once: evict-first
    const float xs[4] = {x.x, x.y, x.z, x.w};
#pragma unroll
    for (int e = 0; e < 4; ++e) {
      const float p = exp2f(fminf(xs[e] + na[i + e] + nbj, 0.f));
#pragma unroll
      for (int r = 0; r < RR; ++r)
        if (r < R) acc[r] = fmaf(p, W[(i + e) * R + r], acc[r]);
    }
  }
  for (int64_t i = M4 + threadIdx.x; i < M; i += kThreads) {
    const float p = exp2f(fminf(__ldcs(g + i) + na[i] + nbj, 0.f));
#pragma unroll
    for (int r = 0; r < RR; ++r)
      if (r < R) acc[r] = fmaf(p, W[i * R + r], acc[r]);
  }
  __shared__ double red[kThreads / 32][kMaxR];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
#pragma unroll
  for (int r = 0; r < RR; ++r) {
    double v = acc[r];
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    if (lane == 0) red[warp][r] = v;
  }
  __syncthreads();
  if (threadIdx.x < R) {
    double v = 0.0;
    for (int w = 0; w < kThreads / 32; ++w) v += red[w][threadIdx.x];
    V[j * R + threadIdx.x] = (float)v;
  }
}

}  // namespace

extern "C" __attribute__((visibility("default"))) int unfused_expw_rows(const float* G, const float* na,
                                                                       const float* nb, const float* W, float* V,
                                                                       int64_t n, int64_t M, int R, void* stream) {
  if (n <= 0) return 0;
  if (R < 1 || R > kMaxR) return (int)cudaErrorInvalidValue;
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  if (R == 1)
    expw_rows_kernel<1><<<(unsigned)n, kThreads, 0, st>>>(G, na, nb, W, V, M, R);
  else if (R <= 4)
    expw_rows_kernel<4><<<(unsigned)n, kThreads, 0, st>>>(G, na, nb, W, V, M, R);
  else
    expw_rows_kernel<kMaxR><<<(unsigned)n, kThreads, 0, st>>>(G, na, nb, W, V, M, R);
  return (int)cudaGetLastError();
}
