// ffma2_microbench.cu -- throughput of the fused kernel's inner-loop shape
// (4x8 half micro-tile: 16 FFMA2 per k with 4 broadcast target scalars and 4
// source pairs read by LDS.128) vs. variants, 1 CTA x 512 threads per SM.
#include <cstdio>
#include <cuda_runtime.h>
typedef unsigned long long f2_t;
__device__ __forceinline__ f2_t bc(float x) { f2_t r; asm("mov.b64 %0, {%1, %1};" : "=l"(r) : "f"(x)); return r; }
__device__ __forceinline__ f2_t ffma2(f2_t a, f2_t b, f2_t c) { f2_t d; asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(d) : "l"(a), "l"(b), "l"(c)); return d; }
__device__ __forceinline__ float lo(f2_t v) { float x, y; asm("mov.b64 {%0, %1}, %2;" : "=f"(x), "=f"(y) : "l"(v)); return x + y; }

#define KP 32
#define REPS 64

// V1: LDS-fed, broadcast b (the kernel's shape)
template <int MODE>
__global__ void __launch_bounds__(512, 1) kern(float* out) {
  __shared__ __align__(16) float sa[KP * 128];
  __shared__ __align__(16) float sb[KP * 256];
  for (int i = threadIdx.x; i < KP * 128; i += 512) sa[i] = 1e-3f * (i & 63);
  for (int i = threadIdx.x; i < KP * 256; i += 512) sb[i] = 1e-3f * (i & 31);
  __syncthreads();
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int tx = (warp & 1) * 8 + ((lane & 1) | ((lane >> 2) & 6));
  const int ty = (warp >> 1) * 4 + ((lane >> 1) & 3);
  f2_t acc[4][4];
  float accs[4][8];
  for (int j = 0; j < 4; ++j) for (int p = 0; p < 4; ++p) acc[j][p] = bc(0.f);
  for (int j = 0; j < 4; ++j) for (int p = 0; p < 8; ++p) accs[j][p] = 0.f;
  for (int r = 0; r < REPS; ++r) {
#pragma unroll
    for (int k = 0; k < KP; ++k) {
      const ulonglong2 a01 = *reinterpret_cast<const ulonglong2*>(sa + k * 128 + 4 * tx);
      const ulonglong2 a23 = *reinterpret_cast<const ulonglong2*>(sa + k * 128 + 64 + 4 * tx);
      const float4 b = *reinterpret_cast<const float4*>(sb + k * 256 + 4 * ty + (r & 1) * 128);
      const f2_t av[4] = {a01.x, a01.y, a23.x, a23.y};
      const float bv[4] = {b.x, b.y, b.z, b.w};
      if (MODE == 0) {
#pragma unroll
        for (int j = 0; j < 4; ++j)
#pragma unroll
          for (int p = 0; p < 4; ++p) acc[j][p] = ffma2(bc(bv[j]), av[p], acc[j][p]);
      } else {
        const float4 x0 = *reinterpret_cast<const float4*>(sa + k * 128 + 4 * tx);
        const float4 x1 = *reinterpret_cast<const float4*>(sa + k * 128 + 64 + 4 * tx);
        const float xs[8] = {x0.x, x0.y, x0.z, x0.w, x1.x, x1.y, x1.z, x1.w};
#pragma unroll
        for (int j = 0; j < 4; ++j)
#pragma unroll
          for (int p = 0; p < 8; ++p) accs[j][p] = fmaf(bv[j], xs[p], accs[j][p]);
      }
    }
  }
  float s = 0;
  for (int j = 0; j < 4; ++j) for (int p = 0; p < 4; ++p) s += lo(acc[j][p]);
  for (int j = 0; j < 4; ++j) for (int p = 0; p < 8; ++p) s += accs[j][p];
  if (s == 1234.5f) out[0] = s;
}

// V2: registers only (no LDS), same FFMA2 pattern
__global__ void __launch_bounds__(512, 1) kern_reg(float* out, float s0) {
  f2_t acc[4][4], av[4];
  float bv[4];
  for (int j = 0; j < 4; ++j) for (int p = 0; p < 4; ++p) acc[j][p] = bc(0.f);
  for (int p = 0; p < 4; ++p) av[p] = bc(s0 + p);
  for (int j = 0; j < 4; ++j) bv[j] = s0 * j + threadIdx.x;
  for (int r = 0; r < REPS * KP; ++r) {
#pragma unroll
    for (int j = 0; j < 4; ++j)
#pragma unroll
      for (int p = 0; p < 4; ++p) acc[j][p] = ffma2(bc(bv[j]), av[p], acc[j][p]);
    bv[r & 3] += 1.0f;  // 1 scalar op per 16 FFMA2
  }
  float s = 0;
  for (int j = 0; j < 4; ++j) for (int p = 0; p < 4; ++p) s += lo(acc[j][p]);
  if (s == 1234.5f) out[0] = s;
}

int main() {
  cudaDeviceProp p; cudaGetDeviceProperties(&p, 0);
  float* out; cudaMalloc(&out, 4);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  const int G = p.multiProcessorCount;
  const double lane_ops = (double)G * 512 * REPS * KP * 32;  // 32 lane-FMAs per k per thread
  for (int v = 0; v < 3; ++v) {
    float best = 1e9;
    for (int rep = 0; rep < 5; ++rep) {
      cudaEventRecord(e0);
      if (v == 0) kern<0><<<G, 512>>>(out);
      else if (v == 1) kern<1><<<G, 512>>>(out);
      else kern_reg<<<G, 512>>>(out, 0.5f);
      cudaEventRecord(e1); cudaEventSynchronize(e1);
      float ms; cudaEventElapsedTime(&ms, e0, e1);
      if (ms < best) best = ms;
    }
    const char* names[] = {"FFMA2 bcast, LDS-fed (kernel shape)", "scalar FFMA, LDS-fed", "FFMA2 bcast, registers only"};
    printf("%-40s %.3f ms  %.1f lane-FMA/clk/SM @1965MHz\n", names[v], best, lane_ops / (best * 1e-3) / G / 1.965e9);
  }
  printf("%s\n", cudaGetErrorString(cudaGetLastError()));
}
