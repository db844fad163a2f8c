// sfu_microbench.cu -- MUFU.EX2 throughput on B200 and whether it overlaps
// the FMA pipe.  32 independent ex2 chains per thread (x = 2^-x, bounded),
// optionally K independent FFMA2 per MUFU; 1 CTA x 512 threads per SM.
#include <cstdio>
#include <cuda_runtime.h>
typedef unsigned long long f2_t;
__device__ __forceinline__ f2_t bc(float x) { f2_t r; asm("mov.b64 %0, {%1, %1};" : "=l"(r) : "f"(x)); return r; }
__device__ __forceinline__ f2_t ffma2(f2_t a, f2_t b, f2_t c) { f2_t d; asm volatile("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(d) : "l"(a), "l"(b), "l"(c)); return d; }
__device__ __forceinline__ float lo(f2_t v) { float x, y; asm("mov.b64 {%0, %1}, %2;" : "=f"(x), "=f"(y) : "l"(v)); return x + y; }
__device__ __forceinline__ float ex2n(float x) { float y; asm volatile("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(-x)); return y; }
#define IT 256
template <int NM, int K>  // per inner step: NM MUFU (of 32 chains) and K*NM... see below
__global__ void __launch_bounds__(512, 1) k(float* out, float s0) {
  float x[32];
  f2_t acc[16];
  for (int i = 0; i < 32; ++i) x[i] = s0 * i * 0.01f;
  for (int i = 0; i < 16; ++i) acc[i] = bc(s0 * i);
  const f2_t a = bc(1.0001f), b = bc(0.999f);
  for (int r = 0; r < IT; ++r) {
#pragma unroll
    for (int i = 0; i < 32; ++i) {
      if (NM) x[i] = ex2n(x[i]);
#pragma unroll
      for (int q = 0; q < K; ++q) acc[(i * K + q) & 15] = ffma2(acc[(i * K + q) & 15], a, b);
    }
  }
  float s = 0.f;
  for (int i = 0; i < 32; ++i) s += x[i];
  for (int i = 0; i < 16; ++i) s += lo(acc[i]);
  if (s == 1234.5f) out[0] = s;
}
template <int NM, int K>
void run(const char* name, float* out, int G, int thr) {
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  float best = 1e9;
  for (int r = 0; r < 5; ++r) {
    cudaEventRecord(e0); k<NM, K><<<G, thr>>>(out, 0.5f); cudaEventRecord(e1); cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1); if (ms < best) best = ms;
  }
  const double warps = (double)G * thr / 32;
  const double steps = (double)IT * 32;  // inner steps per warp
  const double cyc = best * 1e-3 * 1.965e9;  // at sm_max clock
  // cycles per inner step per SMSP: (cyc) / (steps * warps_per_smsp)
  printf("%-40s thr %4d  %.3f ms  %.2f SMSP-cycles per warp-step  (%s)\n", name, thr, best,
         cyc / (steps * warps / G / 4), NM ? "1 MUFU/step" : "no MUFU");
}
int main() {
  cudaDeviceProp p; cudaGetDeviceProperties(&p, 0);
  float* out; cudaMalloc(&out, 4); int G = p.multiProcessorCount;
  for (int thr : {256, 512}) {
    run<1, 0>("MUFU.EX2 only", out, G, thr);
    run<0, 1>("1 FFMA2 only", out, G, thr);
    run<0, 4>("4 FFMA2 only", out, G, thr);
    run<1, 1>("MUFU + 1 FFMA2", out, G, thr);
    run<1, 2>("MUFU + 2 FFMA2", out, G, thr);
    run<1, 4>("MUFU + 4 FFMA2", out, G, thr);
    run<1, 6>("MUFU + 6 FFMA2", out, G, thr);
  }
  printf("%s\n", cudaGetErrorString(cudaGetLastError()));
}
