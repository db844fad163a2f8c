// issue_microbench.cu -- does a warp issuing tcgen05.mma slow the other warps of its SM
// sub-partition?  16 "epilogue" warps (4..19, four per sub-partition) run the R > 1 kernel's
// per-element mix (ex2, split, pack) and store 32 columns to TMEM per iteration; warp 2 (on
// sub-partition 2) issues kind::f16 MMAs (A and B from shared memory, M = 128, N = 96 or ts N = 32)
// into TMEM columns 384+ in batches of B, committing and waiting per batch, until the epilogue
// warps finish.  Reports each sub-partition's mean epilogue finish time (clock64 cycles) and the
// MMA count.
#include <cstdio>
#include <cuda_runtime.h>
#include <cuda_fp16.h>
#include "../paper_conf_icppw_wangkbgj16_b200/csrc/ks_ptx.cuh"
using namespace ks;

constexpr int ITERS = 3000;

template <int B, bool TS>
__global__ void __launch_bounds__(640, 1) k(float* out, int mma_on) {
  extern __shared__ __align__(1024) uint8_t smem[];
  __shared__ uint32_t tb_smem;
  __shared__ __align__(8) uint64_t done;
  __shared__ volatile int stop;
  __shared__ long long fin[20];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (warp == 0) tmem_alloc(&tb_smem, 512);
  if (threadIdx.x == 0) {
    mbar_init(&done, 1);
    stop = 0;
    fence_mbar_init();
  }
  for (int i = threadIdx.x; i < 32768 / 4; i += blockDim.x) reinterpret_cast<uint32_t*>(smem)[i] = 0x30003000u ^ i;
  fence_proxy_async_smem();
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tbase = tb_smem;
  const long long t0 = clock64();
  if (warp >= 4) {
    const int ew = warp - 4, g = ew & 3, slot = ew >> 2;
    const uint32_t ta = tbase + ((uint32_t)(32 * g) << 16) + (uint32_t)(slot * 64);
    uint32_t r[32];
#pragma unroll
    for (int i = 0; i < 32; ++i) r[i] = __float_as_uint(-0.01f * (float)(i + lane));
    for (int it = 0; it < ITERS; ++it) {
      uint32_t o[32];
#pragma unroll
      for (int kk = 0; kk < 16; ++kk) {
        const float t0f = fminf(__uint_as_float(r[2 * kk]), 14.f), t1f = fminf(__uint_as_float(r[2 * kk + 1]), 14.f);
        const float p0 = ex2_approx(t0f), p1 = ex2_approx(t1f);
        const float h0 = __uint_as_float(__float_as_uint(p0) & 0xFFFFE000u);
        const float h1 = __uint_as_float(__float_as_uint(p1) & 0xFFFFE000u);
        const __half2 hv = __floats2half2_rn(h0, h1), lv = __floats2half2_rn(p0 - h0, p1 - h1);
        o[(kk >> 3) * 16 + (kk & 7)] = *reinterpret_cast<const uint32_t*>(&hv);
        o[(kk >> 3) * 16 + 8 + (kk & 7)] = *reinterpret_cast<const uint32_t*>(&lv);
      }
      tmem_st32(ta, o);
#pragma unroll
      for (int i = 0; i < 32; ++i) r[i] = (o[i] & 0x807FFFFFu) | 0xBC000000u;  // keep inputs small negatives
      if ((it & 3) == 3) tmem_wait_st();
    }
    tmem_wait_st();
    if (lane == 0) fin[warp] = clock64() - t0;
  } else if (warp == 2 && mma_on) {
    const uint32_t lead = elect_one() ? 1u : 0u;
    const uint32_t id = TS ? idesc_f16(128, 32) : idesc_f16(128, 96);
    const uint64_t dA = sdesc_k_sw64(smem), dB = sdesc_k_sw64(smem + 16384);
    int n = 0;
    while (!stop) {
      for (int j = 0; j < B; ++j) {
        if (TS)
          { if (lead) mma_f16_ts(tbase + 384u, tbase + 256u + 8u * (j & 7), dB, id, 1u); }
        else
          mma_f16_ss_if(tbase + 384u, dA, dB, id, 1u, lead);
      }
      ++n;
      tc_commit_if(&done, lead);
      mbar_wait(&done, (uint32_t)((n - 1) & 1));
    }
    if (lane == 0 && blockIdx.x == 0) out[8] = (float)n * B;
  }
  if (warp >= 4) {
    asm volatile("bar.sync 1, 512;");
    if (threadIdx.x == 128) stop = 1;
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  if (warp == 0) tmem_dealloc(tbase, 512);
  if (threadIdx.x < 4 && blockIdx.x == 0) {
    double s = 0;
    for (int w = 4; w < 20; ++w)
      if ((w & 3) == threadIdx.x) s += (double)fin[w];
    out[threadIdx.x] = (float)(s / 4.0);
  }
}


template <int B, bool TS>
void run(float* out, int G, int mma_on) {
  auto kern = k<B, TS>;
  cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 40960);
  cudaMemset(out, 0, 64);
  kern<<<G, 640, 40960>>>(out, mma_on);
  kern<<<G, 640, 40960>>>(out, mma_on);
  cudaDeviceSynchronize();
  float h[9];
  cudaMemcpy(h, out, 36, cudaMemcpyDeviceToHost);
  printf("%s B=%2d mma=%d: epilogue finish per sub-partition %8.0f %8.0f %8.0f %8.0f cycles; MMAs %6.0f  %s\n",
         TS ? "ts N=32" : "ss N=96", B, mma_on, h[0], h[1], h[2], h[3], h[8], cudaGetErrorString(cudaGetLastError()));
}

int main() {
  cudaDeviceProp p;
  cudaGetDeviceProperties(&p, 0);
  const int G = p.multiProcessorCount;
  float* out;
  cudaMalloc(&out, 64);
  run<1, false>(out, G, 0);
  run<1, false>(out, G, 1);
  run<4, false>(out, G, 1);
  run<12, false>(out, G, 1);
  run<1, true>(out, G, 1);
  run<12, true>(out, G, 1);
  run<48, true>(out, G, 1);
  printf("%s\n", cudaGetErrorString(cudaDeviceSynchronize()));
}
