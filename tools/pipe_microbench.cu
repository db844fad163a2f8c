// pipe_microbench.cu -- measured per-SM throughput of the instructions the
// fused FP32 kernel is built from (FFMA, FFMA2 = fma.rn.f32x2, MUFU.EX2,
// FMNMX) on this B200.  Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3
#include <cstdio>
#include <cuda_runtime.h>

#define ITERS 4096

__global__ void k_ffma(float* out, float s) {
  float a[16];
#pragma unroll
  for (int i = 0; i < 16; ++i) a[i] = threadIdx.x * 0.001f + i;
  long long t0 = clock64();
  for (int it = 0; it < ITERS; ++it) {
#pragma unroll
    for (int i = 0; i < 16; ++i) a[i] = fmaf(a[i], s, 0.5f * i + 1e-3f);
  }
  float r = 0; for (int i = 0; i < 16; ++i) r += a[i];
  if (r == 12345.f) out[0] = r + (float)(clock64() - t0);
}

__global__ void k_ffma3(float* out, float s, float t) {
  // 3-register form: acc = b * a + acc, like the dot-product inner loop
  float acc[32]; float b[4] = {s, s + 1e-3f, s + 2e-3f, s + 3e-3f};
  float a[8];
#pragma unroll
  for (int i = 0; i < 32; ++i) acc[i] = threadIdx.x * 1e-3f + i;
#pragma unroll
  for (int i = 0; i < 8; ++i) a[i] = t + i * 1e-4f;
  for (int it = 0; it < ITERS / 2; ++it) {
#pragma unroll
    for (int j = 0; j < 4; ++j)
#pragma unroll
      for (int i = 0; i < 8; ++i) acc[j * 8 + i] = fmaf(b[j], a[i], acc[j * 8 + i]);
#pragma unroll
    for (int i = 0; i < 8; ++i) a[i] = a[i] * 0.999f;  // keep a live (8 FMUL per 32 FFMA)
  }
  float r = 0; for (int i = 0; i < 32; ++i) r += acc[i];
  if (r == 12345.f) out[0] = r;
}

__device__ __forceinline__ unsigned long long pack(float x, float y) {
  unsigned long long r;
  asm("mov.b64 %0, {%1, %2};" : "=l"(r) : "f"(x), "f"(y));
  return r;
}
__device__ __forceinline__ void unpack(unsigned long long v, float& x, float& y) {
  asm("mov.b64 {%0, %1}, %2;" : "=f"(x), "=f"(y) : "l"(v));
}
__device__ __forceinline__ unsigned long long ffma2(unsigned long long a, unsigned long long b, unsigned long long c) {
  unsigned long long d;
  asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(d) : "l"(a), "l"(b), "l"(c));
  return d;
}

__global__ void k_ffma2(float* out, float s, float t) {
  unsigned long long acc[16], b[2], a[4];
#pragma unroll
  for (int i = 0; i < 16; ++i) acc[i] = pack(threadIdx.x * 1e-3f + i, i * 0.5f);
  b[0] = pack(s, s + 1e-3f); b[1] = pack(s + 2e-3f, s + 3e-3f);
#pragma unroll
  for (int i = 0; i < 4; ++i) a[i] = pack(t + i * 1e-4f, t - i * 1e-4f);
  for (int it = 0; it < ITERS / 2; ++it) {
#pragma unroll
    for (int j = 0; j < 2; ++j)
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        acc[j * 8 + 2 * i] = ffma2(b[j], a[i], acc[j * 8 + 2 * i]);
        acc[j * 8 + 2 * i + 1] = ffma2(a[i], b[j], acc[j * 8 + 2 * i + 1]);
      }
  }
  float r = 0; for (int i = 0; i < 16; ++i) { float x, y; unpack(acc[i], x, y); r += x + y; }
  if (r == 12345.f) out[0] = r;
}

// outer product with a broadcast scalar operand: acc(j, 2i..2i+1) += b_j * a(2i..2i+1)
__global__ void k_ffma2_bcast(float* out, float s, float t) {
  unsigned long long acc[32], a[4];
  float b[8];
#pragma unroll
  for (int i = 0; i < 32; ++i) acc[i] = pack(threadIdx.x * 1e-3f + i, i * 0.5f);
#pragma unroll
  for (int j = 0; j < 8; ++j) b[j] = s + j * 1e-3f;
#pragma unroll
  for (int i = 0; i < 4; ++i) a[i] = pack(t + i * 1e-4f, t - i * 1e-4f);
  for (int it = 0; it < ITERS / 4; ++it) {
#pragma unroll
    for (int j = 0; j < 8; ++j)
#pragma unroll
      for (int i = 0; i < 4; ++i) acc[j * 4 + i] = ffma2(pack(b[j], b[j]), a[i], acc[j * 4 + i]);
#pragma unroll
    for (int j = 0; j < 8; ++j) b[j] = b[j] * 0.999f;
  }
  float r = 0; for (int i = 0; i < 32; ++i) { float x, y; unpack(acc[i], x, y); r += x + y; }
  if (r == 12345.f) out[0] = r;
}

__global__ void k_ex2(float* out, float s) {
  float a[16];
#pragma unroll
  for (int i = 0; i < 16; ++i) a[i] = -(threadIdx.x * 1e-3f + i * 0.01f);
  for (int it = 0; it < ITERS / 4; ++it) {
#pragma unroll
    for (int i = 0; i < 16; ++i) {
      float y; asm volatile("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(a[i])); a[i] = -y;
    }
  }
  float r = 0; for (int i = 0; i < 16; ++i) r += a[i];
  if (r == 12345.f) out[0] = r;
}

__global__ void k_fmnmx(float* out, float s) {
  float a[16];
#pragma unroll
  for (int i = 0; i < 16; ++i) a[i] = threadIdx.x * 1e-3f + i;
  for (int it = 0; it < ITERS; ++it) {
#pragma unroll
    for (int i = 0; i < 16; ++i) { float x; asm volatile("min.f32 %0, %1, %2;" : "=f"(x) : "f"(a[i]), "f"(s)); a[i] = x; }
  }
  float r = 0; for (int i = 0; i < 16; ++i) r += a[i];
  if (r == 12345.f) out[0] = r;
}

int main() {
  int dev = 0; cudaDeviceProp p; cudaGetDeviceProperties(&p, dev);
  int clk_khz = 0; cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, dev);
  printf("device %s, %d SMs, attr clock %d MHz\n", p.name, p.multiProcessorCount, clk_khz / 1000);
  float* out; cudaMalloc(&out, 4);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  int blocks = p.multiProcessorCount * 4, threads = 256;
  struct { const char* name; double ops_per_thread; int which; } tests[] = {
    {"FFMA (imm addend, 16 chains)", 16.0 * ITERS, 0},
    {"FFMA (3-reg outer product 4x8)", 32.0 * (ITERS / 2), 1},
    {"FFMA2 fma.rn.f32x2 (lane-FMAs)", 32.0 * (ITERS / 2), 2},
    {"FFMA2 broadcast b (lane-FMAs)", 64.0 * (ITERS / 4), 5},
    {"MUFU.EX2", 16.0 * (ITERS / 4), 3},
    {"FMNMX", 16.0 * ITERS, 4},
  };
  for (auto& t : tests) {
    for (int rep = 0; rep < 3; ++rep) {
      cudaEventRecord(e0);
      switch (t.which) {
        case 0: k_ffma<<<blocks, threads>>>(out, 0.9999f); break;
        case 1: k_ffma3<<<blocks, threads>>>(out, 0.9999f, 0.5f); break;
        case 2: k_ffma2<<<blocks, threads>>>(out, 0.9999f, 0.5f); break;
        case 3: k_ex2<<<blocks, threads>>>(out, 0.9999f); break;
        case 4: k_fmnmx<<<blocks, threads>>>(out, 0.9999f); break;
        case 5: k_ffma2_bcast<<<blocks, threads>>>(out, 0.9999f, 0.5f); break;
      }
      cudaEventRecord(e1); cudaEventSynchronize(e1);
      float ms; cudaEventElapsedTime(&ms, e0, e1);
      double ops = t.ops_per_thread * blocks * threads;
      if (rep == 2) {
        double rate = ops / (ms * 1e-3);
        printf("%-34s %8.3f ms  %10.3f T lane-ops/s  = %6.1f per SM per clk at 1965 MHz\n", t.name, ms,
               rate / 1e12, rate / p.multiProcessorCount / 1.965e9);
      }
    }
  }
  printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
