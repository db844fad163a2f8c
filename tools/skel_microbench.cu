// skel_microbench.cu -- latencies behind the synchronisation skeleton of the R = 1 kernel
// (ks_fused_r1.cu) on B200, one 640-thread CTA per SM on every SM:
//   lat_ldtm   tcgen05.ld.32x32b.x32 + tcgen05.wait::ld, one warp, serialised
//   lat_commit tcgen05.commit (no MMA pending) -> mbarrier phase seen by the same warp
//   lat_pingpong  mbarrier arrive in warp A -> try_wait wakes warp B -> arrive back
//   skel       the kernel's skeleton: producer warp (arrive full), MMA warp (wait sempty,
//              wait full, commit empty + sfull), 4 groups x 4 epilogue warps (wait sfull,
//              NLD tcgen05.ld x32 with a wait after each, arrive sempty); no data, no math
// Prints SM cycles (clock64) per iteration / per unit.
#include <cstdio>
#include <cuda_runtime.h>
#include "../paper_conf_icppw_wangkbgj16_b200/csrc/ks_ptx.cuh"
using namespace ks;

constexpr int UNITS = 2000;

template <int MODE, int NLD, int COMMIT>
__global__ void __launch_bounds__(640, 1) k(unsigned long long* out) {
  __shared__ uint32_t tb_smem;
  __shared__ __align__(8) uint64_t full[8], empty[8], sfull[4], sempty[4], pp[2];
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  if (warp == 2) tmem_alloc(&tb_smem, 512);
  if (tid == 0) {
    for (int i = 0; i < 8; ++i) { mbar_init(&full[i], 1); mbar_init(&empty[i], 1); }
    for (int i = 0; i < 4; ++i) { mbar_init(&sfull[i], 1); mbar_init(&sempty[i], 4); }
    mbar_init(&pp[0], 1);
    mbar_init(&pp[1], 1);
    fence_mbar_init();
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tbase = tb_smem;
  long long t0 = clock64();
  long long res = 0;
  if (MODE == 0) {  // LDTM latency
    if (warp == 4) {
      uint32_t r[32], x = 0;
      for (int i = 0; i < UNITS; ++i) {
        tmem_ld32(tbase + (uint32_t)(32 * (i & 3)), r);
        tmem_wait_ld();
        x ^= r[0] ^ r[31];
      }
      res = clock64() - t0;
      if (x == 12345u) out[1] = x;
    }
  } else if (MODE == 1) {  // commit latency (same warp)
    if (warp == 1) {
      for (int i = 0; i < UNITS; ++i) {
        if (elect_one()) tc_commit(&sfull[0]);
        __syncwarp();
        mbar_wait(&sfull[0], (uint32_t)(i & 1));
      }
      res = clock64() - t0;
    }
  } else if (MODE == 2) {  // ping-pong between warps 1 and 4
    if (warp == 1 || warp == 4) {
      const int me = warp == 1 ? 0 : 1;
      for (int i = 0; i < UNITS; ++i) {
        if (me == 0) {
          if (lane == 0) mbar_arrive(&pp[0]);
          mbar_wait(&pp[1], (uint32_t)(i & 1));
        } else {
          mbar_wait(&pp[0], (uint32_t)(i & 1));
          if (lane == 0) mbar_arrive(&pp[1]);
        }
      }
      res = clock64() - t0;
    }
  } else {  // skeleton
    if (warp == 0) {
      int s = 0;
      uint32_t ph = 0;
      for (int q = 0; q < UNITS; ++q) {
        mbar_wait(&empty[s], ph ^ 1u);
        if (lane == 0) mbar_arrive(&full[s]);
        __syncwarp();
        if (++s == 6) { s = 0; ph ^= 1u; }
      }
    } else if (warp == 1) {
      const uint32_t lead = elect_one() ? 1u : 0u;
      int s = 0;
      uint32_t ph = 0;
      for (int q = 0; q < UNITS; ++q) {
        const int bq = q & 3;
        if (q >= 4) mbar_wait(&sempty[bq], (uint32_t)(((q >> 2) - 1) & 1));
        mbar_wait(&full[s], ph);
        tc_fence_after();
        if (COMMIT) {
          tc_commit_if(&empty[s], lead);
          tc_commit_if(&sfull[bq], lead);
        } else {
          if (lead) { mbar_arrive(&empty[s]); mbar_arrive(&sfull[bq]); }
        }
        __syncwarp();
        if (++s == 6) { s = 0; ph ^= 1u; }
      }
      res = clock64() - t0;
    } else if (warp >= 4) {
      const int ew = warp - 4, g = ew & 3, gr = ew >> 2;
      const uint32_t ta = tbase + ((uint32_t)(32 * g) << 16) + (uint32_t)(gr * 128);
      uint32_t x = 0;
      for (int q = gr; q < UNITS; q += 4) {
        mbar_wait(&sfull[gr], (uint32_t)((q >> 2) & 1));
        tc_fence_after();
        uint32_t r[32];
#pragma unroll
        for (int l = 0; l < NLD; ++l) {
          tmem_ld32(ta + 32 * l, r);
          tmem_wait_ld();
          x ^= r[l];
        }
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(&sempty[gr]);
      }
      if (x == 12345u) out[1] = x;
    }
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  if (warp == 2) tmem_dealloc(tbase, 512);
  if (blockIdx.x == 0 && (warp == 1 || (MODE == 0 && warp == 4)) && lane == 0) out[0] = (unsigned long long)res;
}

template <int MODE, int NLD, int COMMIT>
void run(unsigned long long* out, int G, const char* name) {
  k<MODE, NLD, COMMIT><<<G, 640>>>(out);
  cudaDeviceSynchronize();
  k<MODE, NLD, COMMIT><<<G, 640>>>(out);
  cudaError_t e = cudaDeviceSynchronize();
  unsigned long long r = 0;
  cudaMemcpy(&r, out, 8, cudaMemcpyDeviceToHost);
  printf("%-44s %8.1f cycles per %s  (%s)\n", name, (double)r / UNITS, MODE == 3 ? "unit" : "iteration",
         cudaGetErrorString(e));
}

int main() {
  cudaDeviceProp p;
  cudaGetDeviceProperties(&p, 0);
  unsigned long long* out;
  cudaMalloc(&out, 64);
  const int G = p.multiProcessorCount;
  run<0, 0, 0>(out, G, "lat_ldtm (ld.32x32b.x32 + wait::ld)");
  run<1, 0, 0>(out, G, "lat_commit (commit -> wait, same warp)");
  run<2, 0, 0>(out, G, "lat_pingpong (arrive -> wait -> arrive)");
  run<3, 4, 1>(out, G, "skel: 4 LDTM, commits");
  run<3, 4, 0>(out, G, "skel: 4 LDTM, plain arrives");
  run<3, 0, 1>(out, G, "skel: no LDTM, commits");
  run<3, 0, 0>(out, G, "skel: no LDTM, plain arrives");
  run<3, 1, 1>(out, G, "skel: 1 LDTM, commits");
  return 0;
}
