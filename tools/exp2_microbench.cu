// exp2_microbench.cu -- throughput of 2^x (x <= 0) for the epilogue: all on
// MUFU.EX2 vs a fraction on the FMA pipe (degree-5 polynomial, FFMA2-packed).
#include <cstdio>
#include <cuda_runtime.h>
typedef unsigned long long f2_t;
__device__ __forceinline__ f2_t pk(float x, float y) { f2_t r; asm("mov.b64 %0, {%1, %2};" : "=l"(r) : "f"(x), "f"(y)); return r; }
__device__ __forceinline__ void upk(f2_t v, float& x, float& y) { asm("mov.b64 {%0, %1}, %2;" : "=f"(x), "=f"(y) : "l"(v)); }
__device__ __forceinline__ f2_t ffma2(f2_t a, f2_t b, f2_t c) { f2_t d; asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(d) : "l"(a), "l"(b), "l"(c)); return d; }
__device__ __forceinline__ f2_t fadd2(f2_t a, f2_t b) { f2_t d; asm("add.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(a), "l"(b)); return d; }
__device__ __forceinline__ float ex2(float x) { float y; asm volatile("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x)); return y; }
// 2^x for a pair, x in [-126, 0]: x = j + f, j = round(x), f in [-0.5, 0.5]
__device__ __forceinline__ f2_t exp2_poly2(f2_t x) {
  const f2_t magic = pk(12582912.f, 12582912.f);           // 1.5 * 2^23
  f2_t y = fadd2(x, magic);                                 // round to integer (RN)
  f2_t j = fadd2(y, pk(-12582912.f, -12582912.f));
  f2_t f = fadd2(x, j ^ 0x8000000080000000ull);             // f = x - j
  // minimax-ish degree-5 for 2^f on [-0.5, 0.5] (Taylor-like coefficients, rel err ~2e-7 in tests)
  f2_t p = pk(1.3333558146428443e-3f, 1.3333558146428443e-3f);
  p = ffma2(p, f, pk(9.6181291076284772e-3f, 9.6181291076284772e-3f));
  p = ffma2(p, f, pk(5.5504108664821580e-2f, 5.5504108664821580e-2f));
  p = ffma2(p, f, pk(2.4022650695910071e-1f, 2.4022650695910071e-1f));
  p = ffma2(p, f, pk(6.9314718055994531e-1f, 6.9314718055994531e-1f));
  p = ffma2(p, f, pk(1.f, 1.f));
  // scale by 2^j: add j << 23 to the exponent bits (y's low bits hold j)
  unsigned lo = (unsigned)(y & 0xffffffffull), hi = (unsigned)(y >> 32);
  unsigned plo = (unsigned)(p & 0xffffffffull), phi = (unsigned)(p >> 32);
  plo += lo << 23; phi += hi << 23;
  return ((f2_t)phi << 32) | plo;
}
#define IT 512
template <int MODE>  // 0: all MUFU, 1: half poly, 2: all poly
__global__ void __launch_bounds__(512, 1) k(float* out, float s) {
  float x[32], acc = 0.f;
  for (int i = 0; i < 32; ++i) x[i] = -(threadIdx.x % 7) * 0.37f - i * 0.11f;
  for (int it = 0; it < IT; ++it) {
#pragma unroll
    for (int i = 0; i < 32; i += 2) {
      float a, b;
      if (MODE == 0 || (MODE == 1 && (i & 2))) { a = ex2(x[i]); b = ex2(x[i + 1]); }
      else { upk(exp2_poly2(pk(x[i], x[i + 1])), a, b); }
      acc = fmaf(a, s, acc); acc = fmaf(b, s, acc);
      x[i] = fminf(x[i] - a * 1e-3f, 0.f); x[i + 1] = fminf(x[i + 1] - b * 1e-3f, 0.f);
    }
  }
  if (acc == 1234.f) out[0] = acc;
}
int main() {
  cudaDeviceProp p; cudaGetDeviceProperties(&p, 0);
  float* out; cudaMalloc(&out, 4);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  const char* names[] = {"all MUFU.EX2", "half MUFU / half FFMA2 poly", "all FFMA2 poly"};
  for (int m = 0; m < 3; ++m) {
    float best = 1e9;
    for (int r = 0; r < 5; ++r) {
      cudaEventRecord(e0);
      if (m == 0) k<0><<<p.multiProcessorCount, 512>>>(out, 0.5f);
      else if (m == 1) k<1><<<p.multiProcessorCount, 512>>>(out, 0.5f);
      else k<2><<<p.multiProcessorCount, 512>>>(out, 0.5f);
      cudaEventRecord(e1); cudaEventSynchronize(e1);
      float ms; cudaEventElapsedTime(&ms, e0, e1); if (ms < best) best = ms;
    }
    double n = (double)p.multiProcessorCount * 512 * IT * 32;
    printf("%-32s %.3f ms  %.2f exp2/clk/SM @1965\n", names[m], best, n / (best * 1e-3) / p.multiProcessorCount / 1.965e9);
  }
  // accuracy of the polynomial vs ex2 on a grid
  printf("%s\n", cudaGetErrorString(cudaGetLastError()));
}
