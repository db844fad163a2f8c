// tmem_microbench.cu -- tcgen05.ld / tcgen05.st throughput per SM (the R > 1 kernel's epilogue
// reads each S buffer and writes the P split back over it: 2 x 48 KB of TMEM traffic per
// 128 x 96 unit).  One CTA per SM, W warps (4 per SM sub-partition = 16 is the kernel's
// epilogue), each warp looping over its lane quarter's 32 x 32-column blocks.
// Modes: ld (ld + wait), st (st + wait), ldst (ld, wait, st, wait), st4 (4 st then one wait),
//        idle (MMA rate alone); with mma=1 warp W keeps the tensor pipe busy with M=128 N=96
//        MMAs meanwhile (its MMA count shows how much the TMEM traffic slows the tensor pipe).
// Reports bytes / clk / SM (clock64 of CTA 0) and ns per 32x32 block per warp.
#include <cstdio>
#include <cuda_runtime.h>
#include <cuda_fp16.h>
#include "../paper_conf_icppw_wangkbgj16_b200/csrc/ks_ptx.cuh"
using namespace ks;

constexpr int ITERS = 4000;

template <int MODE, int W, bool MMA>
__global__ void __launch_bounds__(W * 32 + 64, 1) k(float* out) {
  extern __shared__ __align__(1024) uint8_t smem[];
  __shared__ uint32_t tb_smem;
  __shared__ __align__(8) uint64_t done;
  __shared__ volatile int stop;
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
  long long t0 = clock64();
  if (warp < W) {
    const int g = warp & 3, slot = warp >> 2;  // lane quarter, column block
    const uint32_t ta = tbase + ((uint32_t)(32 * g) << 16) + (uint32_t)((slot * 32) % 384);
    uint32_t r[32];
#pragma unroll
    for (int i = 0; i < 32; ++i) r[i] = 0x3c003c00u + i + lane;
    for (int it = 0; it < ITERS; ++it) {
      if (MODE == 0) {
        tmem_ld32(ta, r);
        tmem_wait_ld();
        r[0] += r[31];
      } else if (MODE == 1) {
        tmem_st32(ta, r);
        tmem_wait_st();
        r[0] += 1;
      } else if (MODE == 2) {
        tmem_ld32(ta, r);
        tmem_wait_ld();
        r[0] += r[31];
        tmem_st32(ta, r);
        tmem_wait_st();
      } else if (MODE == 3) {
        tmem_st32(ta, r);
        r[0] += 1;
        if ((it & 3) == 3) tmem_wait_st();
      } else if (MODE >= 5 && MODE <= 7) {  // 5: 32 MUFU.EX2; 6: st32; 7: both (the epilogue's mix)
        if (MODE != 6) {
#pragma unroll
          for (int i = 0; i < 32; ++i) r[i] = __float_as_uint(ex2_approx(__uint_as_float(r[i])));
        }
        if (MODE != 5) tmem_st32(ta, r);
        if (MODE != 5 && (it & 3) == 3) tmem_wait_st();
      } else if (MODE == 8) {  // 8: the epilogue's full mix per 32 elements (fmin, ex2, split, pack) + st32
        uint32_t o[32];
#pragma unroll
        for (int k = 0; k < 16; ++k) {
          const float t0 = fminf(__uint_as_float(r[2 * k]), 14.f), t1 = fminf(__uint_as_float(r[2 * k + 1]), 14.f);
          const float p0 = ex2_approx(t0), p1 = ex2_approx(t1);
          const float h0 = __uint_as_float(__float_as_uint(p0) & 0xFFFFE000u);
          const float h1 = __uint_as_float(__float_as_uint(p1) & 0xFFFFE000u);
          const __half2 hv = __floats2half2_rn(h0, h1), lv = __floats2half2_rn(p0 - h0, p1 - h1);
          o[(k >> 3) * 16 + (k & 7)] = *reinterpret_cast<const uint32_t*>(&hv);
          o[(k >> 3) * 16 + 8 + (k & 7)] = *reinterpret_cast<const uint32_t*>(&lv);
        }
        if (MODE == 8) tmem_st32(ta, o);
#pragma unroll
        for (int i = 0; i < 32; ++i) r[i] = o[i] ^ (uint32_t)it;
        if ((it & 3) == 3) tmem_wait_st();
      } else if (MODE == 9) {  // 9: mode 8 without the st
        uint32_t o[32];
#pragma unroll
        for (int k = 0; k < 16; ++k) {
          const float t0 = fminf(__uint_as_float(r[2 * k]), 14.f), t1 = fminf(__uint_as_float(r[2 * k + 1]), 14.f);
          const float p0 = ex2_approx(t0), p1 = ex2_approx(t1);
          const float h0 = __uint_as_float(__float_as_uint(p0) & 0xFFFFE000u);
          const float h1 = __uint_as_float(__float_as_uint(p1) & 0xFFFFE000u);
          const __half2 hv = __floats2half2_rn(h0, h1), lv = __floats2half2_rn(p0 - h0, p1 - h1);
          o[(k >> 3) * 16 + (k & 7)] = *reinterpret_cast<const uint32_t*>(&hv);
          o[(k >> 3) * 16 + 8 + (k & 7)] = *reinterpret_cast<const uint32_t*>(&lv);
        }
#pragma unroll
        for (int i = 0; i < 32; ++i) r[i] = o[i] ^ (uint32_t)it;
      } else {  // MODE 4: idle for as long as the st loop takes (MMA rate alone)
        const long long e = t0 + 320000;
        while (clock64() < e) {
        }
        break;
      }
    }
    if (warp == 0 && lane == 0) out[1] = (float)r[0];
  } else if (MMA && warp == W) {
    const uint32_t lead = elect_one() ? 1u : 0u;
    const uint32_t id = idesc_f16(128, 96);
    const uint64_t dA = sdesc_k_sw64(smem), dB = sdesc_k_sw64(smem + 16384);
    int n = 0;
    while (!stop) {
      for (int j = 0; j < 8; ++j) mma_f16_ss_if(tbase + 384u, dA, dB, id, 1u, lead);
      ++n;
      tc_commit_if(&done, lead);
      mbar_wait(&done, (uint32_t)((n - 1) & 1));
    }
    if (lane == 0 && blockIdx.x == 0) out[2] = (float)n;
  }
  long long t1 = clock64();
  if (warp < W) {
    // the compute warps are done: stop the MMA warp
    asm volatile("bar.sync 1, %0;" ::"r"(W * 32));
    if (threadIdx.x == 0) stop = 1;
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  if (warp == 0) tmem_dealloc(tbase, 512);
  if (threadIdx.x == 0 && blockIdx.x == 0) out[0] = (float)(t1 - t0);
}

template <int MODE, int W, bool MMA>
void run(const char* name, float* out, int G) {
  auto kern = k<MODE, W, MMA>;
  cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 40960);
  kern<<<G, W * 32 + 64, 40960>>>(out);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaEventRecord(e0);
  kern<<<G, W * 32 + 64, 40960>>>(out);
  cudaEventRecord(e1);
  cudaEventSynchronize(e1);
  float ms;
  cudaEventElapsedTime(&ms, e0, e1);
  float h[3];
  cudaMemcpy(h, out, 12, cudaMemcpyDeviceToHost);
  const double bytes = (double)W * ITERS * 4096.0 * (MODE == 2 ? 2 : 1);
  printf("%-10s W=%2d mma=%d: %8.0f cycles  %6.1f B/clk/SM  %6.1f cycles per 4 KB block per warp  (%.3f ms, mma iters %.0f) %s\n",
         name, W, MMA ? 1 : 0, h[0], bytes / h[0], h[0] / ITERS / (MODE == 2 ? 2 : 1), ms, MMA ? h[2] : 0.f,
         cudaGetErrorString(cudaGetLastError()));
}

int main() {
  cudaDeviceProp p;
  cudaGetDeviceProperties(&p, 0);
  const int G = p.multiProcessorCount;
  float* out;
  cudaMalloc(&out, 64);
  run<0, 4, false>("ld", out, G);
  run<0, 8, false>("ld", out, G);
  run<0, 16, false>("ld", out, G);
  run<1, 4, false>("st", out, G);
  run<1, 8, false>("st", out, G);
  run<1, 16, false>("st", out, G);
  run<3, 16, false>("st4", out, G);
  run<2, 16, false>("ldst", out, G);
  run<0, 16, true>("ld", out, G);
  run<1, 16, true>("st", out, G);
  run<2, 16, true>("ldst", out, G);
  run<4, 16, true>("idle", out, G);
  run<5, 16, false>("mufu32", out, G);
  run<6, 16, false>("st32", out, G);
  run<7, 16, false>("mufu+st", out, G);
  run<9, 16, false>("epi", out, G);
  run<8, 16, false>("epi+st", out, G);
  run<9, 8, false>("epi", out, G);
  run<8, 8, false>("epi+st", out, G);
  printf("%s\n", cudaGetErrorString(cudaDeviceSynchronize()));
}
