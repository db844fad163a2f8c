// mbar_microbench.cu -- latency of an mbarrier wait on an already-completed
// phase, as seen by one warp in a loop (B200): try_wait (acquire, the default),
// test_wait, try_wait.relaxed, with and without a tcgen05.mma in flight.
// Prints SM cycles per loop iteration at 1965 MHz.
#include <cstdio>
#include <cuda_runtime.h>
#include "../paper_conf_icppw_wangkbgj16_b200/csrc/ks_ptx.cuh"
using namespace ks;
#define ITERS 8192

__device__ __forceinline__ bool try_wait_relaxed(uint32_t bar, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "mbarrier.try_wait.parity.relaxed.cta.shared::cta.b64 p, [%1], %2;\n\t"
      "selp.u32 %0, 1, 0, p;\n\t}"
      : "=r"(ok)
      : "r"(bar), "r"(parity)
      : "memory");
  return ok != 0;
}

// MODE 0 try_wait, 1 test_wait, 2 try_wait.relaxed, 3 try_wait + 1 MMA per iteration,
// 4 test_wait + 1 MMA, 5 relaxed + 1 MMA, 6 two try_waits on different barriers
template <int MODE>
__global__ void __launch_bounds__(128, 1) k(float* out) {
  extern __shared__ __align__(1024) uint8_t smem[];
  __shared__ uint32_t tb;
  __shared__ __align__(8) uint64_t done[2];
  __shared__ __align__(8) uint64_t bar;
  const int tid = threadIdx.x, warp = tid >> 5;
  for (int i = tid; i < 384 * 64 / 4; i += blockDim.x) reinterpret_cast<uint32_t*>(smem)[i] = 0u;
  if (tid == 0) {
    mbar_init(&done[0], 1);
    mbar_init(&done[1], 1);
    mbar_init(&bar, 1);
    fence_mbar_init();
  }
  if (warp == 0) tmem_alloc(&tb, 512);
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  if (tid == 0) {
    mbar_arrive(&done[0]);
    mbar_arrive(&done[1]);
  }
  __syncthreads();
  const uint32_t tbase = tb;
  if (warp == 0) {
    const bool leader = elect_one();
    const uint64_t dA = sdesc_k_sw64(smem), dB = sdesc_k_sw64(smem + 128 * 64);
    const uint32_t id = idesc_f16(128, 256);
    const uint32_t a0 = smem_u32(&done[0]), a1 = smem_u32(&done[1]);
    unsigned long long t0 = clock64();
    for (int i = 0; i < ITERS; ++i) {
      if (MODE >= 3 && MODE <= 5) {
        if (leader) mma_f16_ss(tbase + (uint32_t)((i & 1) * 256), dA, dB, id, 0u);
        __syncwarp();
      }
      if (MODE == 0 || MODE == 3 || MODE == 6) while (!mbar_try_wait(a0, 0)) {}
      if (MODE == 6) while (!mbar_try_wait(a1, 0)) {}
      if (MODE == 1 || MODE == 4) while (!mbar_test(&done[0], 0)) {}
      if (MODE == 2 || MODE == 5) while (!try_wait_relaxed(a0, 0)) {}
    }
    if (leader) tc_commit(&bar);
    __syncwarp();
    mbar_wait(&bar, 0);
    unsigned long long t1 = clock64();
    if (tid == 0 && blockIdx.x == 0) out[0] = (float)(t1 - t0) / ITERS;
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 0) tmem_dealloc(tbase, 512);
}

template <int MODE>
void run(const char* name, float* out, int G) {
  const int smem = 384 * 64 + 1024;
  cudaFuncSetAttribute(k<MODE>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  k<MODE><<<G, 128, smem>>>(out);
  cudaDeviceSynchronize();
  float c;
  cudaMemcpy(&c, out, 4, cudaMemcpyDeviceToHost);
  printf("%-40s %.1f SM cycles per iteration (clock64)\n", name, c);
}
int main() {
  cudaDeviceProp p;
  cudaGetDeviceProperties(&p, 0);
  float* out;
  cudaMalloc(&out, 8);
  const int G = p.multiProcessorCount;
  run<0>("try_wait (acquire), completed", out, G);
  run<1>("test_wait, completed", out, G);
  run<2>("try_wait.relaxed, completed", out, G);
  run<3>("1 MMA + try_wait", out, G);
  run<4>("1 MMA + test_wait", out, G);
  run<5>("1 MMA + try_wait.relaxed", out, G);
  run<6>("two try_waits", out, G);
  printf("%s\n", cudaGetErrorString(cudaDeviceSynchronize()));
}
