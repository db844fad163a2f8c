// lds_microbench.cu -- shared-memory load throughput on B200 by width and
// address pattern (how many distinct 16-byte chunks a warp touches).
#include <cstdio>
#include <cuda_runtime.h>
#define N_IT 2048
template <int W, int PAT>
__global__ void __launch_bounds__(512, 1) k(float* out) {
  __shared__ __align__(16) float s[8192];
  for (int i = threadIdx.x; i < 8192; i += 512) s[i] = i * 1e-4f;
  __syncthreads();
  const int lane = threadIdx.x & 31;
  int off;
  if (PAT == 0) off = 0;                                                   // all lanes same chunk
  else if (PAT == 1) off = ((lane >> 1) & 3) * 4;                          // 4 chunks (kernel's target load)
  else if (PAT == 2) off = ((lane & 1) | ((lane >> 2) & 6)) * 4;           // 8 chunks (kernel's source load)
  else if (PAT == 3) off = (lane & 7) * 4;                                 // 8 chunks, lane-contiguous quarters
  else off = lane * 4;                                                     // 32 distinct chunks
  float acc0 = 0, acc1 = 0, acc2 = 0, acc3 = 0;
  const float* p = s + off + (threadIdx.x >> 5) * 128;
#pragma unroll 16
  for (int it = 0; it < N_IT; ++it) {
    const float* q = p + (it & 7) * 512;
    const unsigned a = (unsigned)__cvta_generic_to_shared(q);
    if (W == 16) { float x, y, z, w; asm volatile("ld.shared.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(x), "=f"(y), "=f"(z), "=f"(w) : "r"(a)); acc0 += x; acc1 += y; acc2 += z; acc3 += w; }
    else if (W == 8) { float x, y; asm volatile("ld.shared.v2.f32 {%0,%1}, [%2];" : "=f"(x), "=f"(y) : "r"(a)); acc0 += x; acc1 += y; }
    else { float x; asm volatile("ld.shared.f32 %0, [%1];" : "=f"(x) : "r"(a)); acc0 += x; }
  }
  if (acc0 + acc1 + acc2 + acc3 == 1234.f) out[0] = acc0;
}
template <int W, int PAT>
void run(const char* name, int G, float* out) {
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  float best = 1e9;
  for (int r = 0; r < 5; ++r) {
    cudaEventRecord(e0); k<W, PAT><<<G, 512>>>(out); cudaEventRecord(e1); cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1); if (ms < best) best = ms;
  }
  double warp_lds = (double)16 * N_IT;  // per SM
  double cyc = best * 1e-3 * 1.965e9;
  printf("LDS.%-3d %-38s %.3f ms  %.2f cycles per warp-LDS per SM  (%.0f B/clk to registers)\n", W * 8, name, best,
         cyc / warp_lds, warp_lds * 32 * W / cyc);
}
int main() {
  cudaDeviceProp p; cudaGetDeviceProperties(&p, 0);
  float* out; cudaMalloc(&out, 4);
  int G = p.multiProcessorCount;
  run<16, 0>("1 chunk (full broadcast)", G, out);
  run<16, 1>("4 chunks (target pattern)", G, out);
  run<16, 2>("8 chunks (source pattern, new map)", G, out);
  run<16, 3>("8 chunks (lane&7)", G, out);
  run<16, 4>("32 chunks", G, out);
  run<8, 0>("1 chunk", G, out);
  run<8, 1>("4 chunks", G, out);
  run<8, 4>("32 chunks", G, out);
  run<4, 0>("1 word", G, out);
  run<4, 4>("32 words", G, out);
  printf("%s\n", cudaGetErrorString(cudaGetLastError()));
}
