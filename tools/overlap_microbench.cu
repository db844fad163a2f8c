// overlap_microbench.cu -- do MUFU.EX2 and the FP32 (FMA) pipe overlap on B200?
// 1 CTA x 512 threads per SM (4 warps per SMSP).  Per loop iteration each
// thread issues NF independent FFMA2 (or FADD2 / scalar FFMA) and NM independent
// MUFU.EX2 (8 self-chains, ex2(-y)); MUFU results are consumed by the chains
// only, FMA results by their own accumulators.  Prints SMSP cycles per iteration
// per warp at 1965 MHz; compare with the sum and the max of the pure cases.
#include <cstdio>
#include <cuda_runtime.h>
typedef unsigned long long f2_t;
__device__ __forceinline__ f2_t bc(float x) {
  f2_t r;
  asm("mov.b64 %0, {%1, %1};" : "=l"(r) : "f"(x));
  return r;
}
__device__ __forceinline__ f2_t ffma2(f2_t a, f2_t b, f2_t c) {
  f2_t d;
  asm volatile("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(d) : "l"(a), "l"(b), "l"(c));
  return d;
}
__device__ __forceinline__ f2_t fadd2(f2_t a, f2_t b) {
  f2_t d;
  asm volatile("add.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(a), "l"(b));
  return d;
}
__device__ __forceinline__ float ex2n(float x) {
  float y;
  asm volatile("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(-x));
  return y;
}
__device__ __forceinline__ float ffma1(float a, float b, float c) {
  float d;
  asm volatile("fma.rn.f32 %0, %1, %2, %3;" : "=f"(d) : "f"(a), "f"(b), "f"(c));
  return d;
}
#define IT 4096
// KIND 0: FFMA2, 1: FADD2, 2: scalar FFMA
template <int NF, int NM, int KIND>
__global__ void __launch_bounds__(512, 1) k(float* out, float s0) {
  f2_t acc[16];
  float accs[16];
  float y[8];
  const f2_t b2 = bc(s0), c2 = bc(1.0f + s0);
#pragma unroll
  for (int i = 0; i < 16; ++i) { acc[i] = bc(s0 * i); accs[i] = s0 * i; }
#pragma unroll
  for (int i = 0; i < 8; ++i) y[i] = 0.1f * i + s0 * threadIdx.x;
  for (int r = 0; r < IT; ++r) {
#pragma unroll
    for (int i = 0; i < 16; ++i) {
      if (i < NF) {
        if (KIND == 0) acc[i] = ffma2(acc[i], b2, c2);
        else if (KIND == 1) acc[i] = fadd2(acc[i], c2);
        else accs[i] = ffma1(accs[i], s0, 1.0f);
      }
      if (i < NM) y[i & 7] = ex2n(y[i & 7]);
    }
  }
  float s = 0.f;
#pragma unroll
  for (int i = 0; i < 16; ++i) {
    float a, b;
    asm("mov.b64 {%0, %1}, %2;" : "=f"(a), "=f"(b) : "l"(acc[i]));
    s += a + b + accs[i];
  }
#pragma unroll
  for (int i = 0; i < 8; ++i) s += y[i];
  if (s == 1234.5f) out[0] = s;
}
template <int NF, int NM, int KIND>
void run(float* out, int G) {
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  float best = 1e9;
  for (int r = 0; r < 5; ++r) {
    cudaEventRecord(e0);
    k<NF, NM, KIND><<<G, 512>>>(out, 0.5f);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    if (ms < best) best = ms;
  }
  // 4 warps per SMSP: cycles per iteration per warp
  const double cyc = best * 1e-3 * 1.965e9 / IT / 4;
  const char* kn = KIND == 0 ? "FFMA2" : KIND == 1 ? "FADD2" : "FFMA ";
  printf("%2d %s + %2d MUFU.EX2 per iter: %.3f ms  %6.2f SMSP cycles/iter/warp\n", NF, kn, NM, best, cyc);
}
int main() {
  cudaDeviceProp p;
  cudaGetDeviceProperties(&p, 0);
  float* out;
  cudaMalloc(&out, 4);
  const int G = p.multiProcessorCount;
  run<0, 8, 0>(out, G);
  run<0, 16, 0>(out, G);
  run<16, 0, 0>(out, G);
  run<8, 0, 0>(out, G);
  run<16, 0, 1>(out, G);
  run<16, 0, 2>(out, G);
  run<16, 4, 0>(out, G);
  run<16, 8, 0>(out, G);
  run<8, 8, 0>(out, G);
  run<4, 8, 0>(out, G);
  run<2, 8, 0>(out, G);
  run<8, 8, 1>(out, G);
  run<4, 8, 1>(out, G);
  run<16, 8, 2>(out, G);
  run<8, 8, 2>(out, G);
  run<4, 8, 2>(out, G);
  printf("%s\n", cudaGetErrorString(cudaDeviceSynchronize()));
}
