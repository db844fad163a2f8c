// epi_microbench.cu -- the R=1 log-weight epilogue of ks_fused_tc_kernel in
// isolation: 16 compute warps (+3 idle) per SM, 1 CTA/SM, 900 "tiles" of
// 64 elements per thread; S from TMEM (tcgen05.ld) or from registers.
// Reports SMSP cycles per warp-element (MUFU.EX2 bound = ~8.4).
#include <cstdio>
#include <cstdlib>
#include <cuda_runtime.h>
#include "../paper_conf_icppw_wangkbgj16_b200/csrc/ks_ptx.cuh"
using namespace ks;
#define TILES 900
__device__ __forceinline__ bool try_wait_hint(uint32_t bar, uint32_t parity, uint32_t ns) {
  uint32_t ok;
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n\t"
      "selp.u32 %0, 1, 0, p;\n\t}"
      : "=r"(ok)
      : "r"(bar), "r"(parity), "r"(ns)
      : "memory");
  return ok != 0;
}
// SPIN: warps 0, 1, 3 wait on a barrier the compute warps complete at the end:
// 0 none, 1 try_wait loop, 2 try_wait with suspend hint, 3 test_wait + nanosleep(64)
template <int MODE, int BC, int SPIN = 0>
__global__ void __launch_bounds__(640, 1) k(float* out, float s0) {
  __shared__ __align__(16) float nas[2][256];
  __shared__ uint32_t tb_smem;
  __shared__ __align__(8) uint64_t done_bar;
  if (threadIdx.x == 0) { mbar_init(&done_bar, 16); fence_mbar_init(); }
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  for (int i = tid; i < 512; i += blockDim.x) nas[i >> 8][i & 255] = -0.01f * (i & 255);
  if (warp == 2) tmem_alloc(&tb_smem, 512);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tbase = tb_smem;
  if (SPIN && (warp == 0 || warp == 1 || warp == 3)) {
    const uint32_t a = smem_u32(&done_bar);
    if (SPIN == 1) { while (!mbar_try_wait(a, 0)) {} }
    else if (SPIN == 2) { while (!try_wait_hint(a, 0, 1000000u)) {} }
    else { while (!mbar_test(&done_bar, 0)) __nanosleep(64); }
  }
  if (warp >= 4) {
    const int ew = warp - 4, g = ew & 3, h = ew >> 2;
    const uint32_t lane_off = (uint32_t)(32 * g) << 16;
    f2_t acc[2] = {0ull, 0ull};
    const f2_t nb2 = f2_bcast(-0.5f * s0), rj2 = f2_bcast(s0);
    for (int q = 0; q < TILES; ++q) {
      const float* na = nas[q & 1];
#pragma unroll
      for (int hh = 0; hh < 64 / BC; ++hh) {
        const int c0 = 64 * h + BC * hh;
        uint32_t sv[BC];
        if (MODE == 1) {
          tmem_ldn<BC>(tbase + lane_off + (q & 1) * 256 + c0, sv);
          tmem_wait_ld();
        } else {
#pragma unroll
          for (int e = 0; e < BC; ++e) sv[e] = __float_as_uint(-0.001f * (float)(e + q + lane));
        }
#pragma unroll
        for (int i = 0; i < BC; i += 4) {
          const ulonglong2 na2 = lds_pairs(na + c0 + i);
#pragma unroll
          for (int u = 0; u < 2; ++u) {
            const f2_t x = ffma2f(f2_pack(__uint_as_float(sv[i + 2 * u]), __uint_as_float(sv[i + 2 * u + 1])), rj2,
                                  fadd2(u ? na2.y : na2.x, nb2));
            float t0, t1;
            f2_unpack(x, t0, t1);
            acc[u] = fadd2(acc[u], f2_pack(ex2_approx(t0), ex2_approx(t1)));
          }
        }
      }
    }
    float a, b, c, d;
    f2_unpack(acc[0], a, b);
    f2_unpack(acc[1], c, d);
    if (a + b + c + d == 1234.5f) out[0] = a;
    __syncwarp();
    if (lane == 0) mbar_arrive(&done_bar);
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 2) tmem_dealloc(tbase, 512);
}
template <int MODE, int BC, int SPIN = 0>
void run(const char* name, float* out, int G) {
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  float best = 1e9;
  for (int r = 0; r < 5; ++r) {
    cudaEventRecord(e0); k<MODE, BC, SPIN><<<G, 640>>>(out, 0.5f); cudaEventRecord(e1); cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1); if (ms < best) best = ms;
  }
  const double elem_warps_per_smsp = (double)TILES * 64 * 4;  // 4 compute warps per SMSP
  printf("%-36s %.3f ms  %.2f SMSP-cycles per warp-element @1965\n", name, best,
         best * 1e-3 * 1.965e9 / elem_warps_per_smsp);
}
int main(int argc, char** argv) {
  cudaDeviceProp p; cudaGetDeviceProperties(&p, 0);
  float* out; cudaMalloc(&out, 4); int G = p.multiProcessorCount;
  const int v = argc > 1 ? atoi(argv[1]) : 0;
  switch (v) {
    case 0: run<0, 32>("registers, BC 32", out, G); break;
    case 1: run<1, 32>("tcgen05.ld x32 + wait, BC 32", out, G); break;
    case 2: run<1, 16>("tcgen05.ld x16 + wait, BC 16", out, G); break;
    case 3: run<1, 32, 1>("ld x32, 3 warps try_wait spinning", out, G); break;
    case 4: run<1, 32, 2>("ld x32, 3 warps try_wait+hint", out, G); break;
    case 5: run<1, 32, 3>("ld x32, 3 warps test+nanosleep", out, G); break;
  }
  printf("%s\n", cudaGetErrorString(cudaDeviceSynchronize()));
  fflush(stdout);
}
