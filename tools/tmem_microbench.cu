// tmem_microbench.cu -- TMEM read bandwidth and its interaction with MUFU.EX2
// on one B200 SM (1 CTA/SM, 16 reader warps = 4 per SMSP, like the fused
// kernel's epilogue).  Reports bytes per SM clock (at 1965 MHz) and elements
// per SM clock.  Question it answers: does tcgen05.ld (4 B per kernel value)
// cap the R=1 epilogue below the MUFU.EX2 rate of 16/clk/SM?
#include <cstdio>
#include <cstdlib>
#include <cuda_runtime.h>
#include "../paper_conf_icppw_wangkbgj16_b200/csrc/ks_ptx.cuh"
using namespace ks;
#define ITERS 4000

__device__ __forceinline__ void ld16x256_x8(uint32_t a, uint32_t (&r)[32]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.16x256b.x8.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
      "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
        "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]),
        "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]),
        "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
      : "r"(a));
}

// MODE 0: 32x32b.x32 loads only (xor-reduce), 1: 16x256b.x8 loads only,
// 2: 32x32b.x32 + one ex2 per element, 3: registers (no TMEM) + one ex2 per element,
// 4: two 32x32b.x32 loads in flight before one wait
template <int MODE>
__global__ void __launch_bounds__(640, 1) k(float* out, int nwarps) {
  __shared__ uint32_t tb_smem;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  if (warp == 0) tmem_alloc(&tb_smem, 512);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tbase = tb_smem;
  if (warp >= 4 && warp < 4 + nwarps) {
    const int ew = warp - 4, g = ew & 3, h = ew >> 2;
    const uint32_t lane_off = (uint32_t)(32 * g) << 16;
    uint32_t x = 0;
    f2_t acc = 0ull;
    for (int q = 0; q < ITERS; ++q) {
      const uint32_t col = (uint32_t)((q * 32 + h * 128) & 511);
      uint32_t sv[32];
      if (MODE == 0 || MODE == 2) {
        tmem_ld32(tbase + lane_off + col, sv);
        tmem_wait_ld();
      } else if (MODE == 1) {
        ld16x256_x8(tbase + lane_off + (col & 448), sv);
        tmem_wait_ld();
      } else if (MODE == 4) {
        uint32_t sw[32];
        tmem_ld32(tbase + lane_off + col, sv);
        tmem_ld32(tbase + lane_off + ((col + 256) & 511), sw);
        tmem_wait_ld();
#pragma unroll
        for (int i = 0; i < 32; ++i) x ^= sw[i];
        ++q;
      } else {
#pragma unroll
        for (int i = 0; i < 32; ++i) sv[i] = __float_as_uint(-0.001f * (float)(i + q + lane));
      }
      if (MODE == 2 || MODE == 3) {
#pragma unroll
        for (int i = 0; i < 32; i += 2)
          acc = fadd2(acc, f2_pack(ex2_approx(-__uint_as_float(sv[i] & 0x3fffffffu)),
                                   ex2_approx(-__uint_as_float(sv[i + 1] & 0x3fffffffu))));
      } else {
#pragma unroll
        for (int i = 0; i < 32; ++i) x ^= sv[i];
      }
    }
    float a, b;
    f2_unpack(acc, a, b);
    if (x == 0x12345u || a + b == 1234.5f) out[0] = a + (float)x;
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 0) tmem_dealloc(tbase, 512);
}

template <int MODE>
void run(const char* name, float* out, int G, int nw) {
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  float best = 1e9;
  for (int r = 0; r < 5; ++r) {
    cudaEventRecord(e0);
    k<MODE><<<G, 640>>>(out, nw);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    if (ms < best) best = ms;
  }
  const double elems_per_sm = (double)ITERS * 32 * 32 * nw;  // 32 columns x 32 lanes per warp-load
  const double clk = best * 1e-3 * 1.965e9;
  printf("%-44s warps %2d  %.3f ms  %.1f elem/clk/SM  %.1f B/clk/SM\n", name, nw, best, elems_per_sm / clk,
         4 * elems_per_sm / clk);
}

int main() {
  cudaDeviceProp p;
  cudaGetDeviceProperties(&p, 0);
  float* out;
  cudaMalloc(&out, 4);
  const int G = p.multiProcessorCount;
  for (int nw : {4, 8, 16}) {
    run<0>("tcgen05.ld 32x32b.x32 + wait", out, G, nw);
    run<4>("2x tcgen05.ld 32x32b.x32 + one wait", out, G, nw);
    run<1>("tcgen05.ld 16x256b.x8 + wait", out, G, nw);
    run<2>("tcgen05.ld 32x32b.x32 + ex2 each", out, G, nw);
    run<3>("registers + ex2 each", out, G, nw);
  }
  printf("%s\n", cudaGetErrorString(cudaDeviceSynchronize()));
}
