// ks_fused_fp32.cu -- the fused FP32 kernel-summation kernel (scope rows a2-a7)
// for K <= 32, R = 1.
//
// What it computes (PAPER.md SS III-C, Alg.2, with Eq.3):
// for every target j,  V_j = sum_i ex2(min(t_ij, 0)) * W_i  with
//   t_ij = sum_d a_id * bh_jd + na_i + nb_j
//        = 2c a_hat_i.b_hat_j - c||a_hat_i||^2 - c||b_hat_j||^2
//        = -log2(e) ||alpha_i - beta_j||^2 / (2h^2)
// so ex2(t_ij) = exp(-||alpha_i - beta_j||^2 / 2h^2) (Eq.1) and the sum is Eq.2.
// The clamp min(t, 0) is d^2 >= 0 (north_star; reading Q8).
//
// B200 design (SS6), not the paper's Maxwell one:
//  * one persistent 512-thread CTA per SM over a stream-K split of the
//    (256-target tile x 128-source tile) unit space -> no wave quantisation
//    and no co-resident CTAs racing each other (the warp arbiter is not fair
//    between CTAs; a lone slow CTA left on an SM idles half its pipes);
//  * the CTA's 256-target tile lives in shared memory for the whole segment
//    (centred and normed in the prologue = row a2, Alg.1 l.4 P:L118-120);
//  * 128-source tiles [k_pad + 2][128] (prescaled coordinates, norms, W) are
//    streamed by TMA into an S-stage mbarrier ring (replaces the paper's
//    double buffering, Alg.2 l.5-11 P:L248-256); the last warp to release a
//    stage issues its refill (no producer warp, nobody waits);
//  * each thread owns an 8x8 register micro-tile (8 targets x 8 sources,
//    the paper's 8x8 microtile P:L168) as two 4x8 halves; the contraction
//    uses packed FFMA2 (fma.rn.f32x2: two FP32 FMAs per issue slot, the
//    target coordinate as a broadcast operand) fed by LDS.128 whose lane
//    mapping keeps each quarter-warp on <= 64 B (2 wavefronts per load);
//  * epilogue (Alg.2 l.14-16 P:L258-260) of one half -- FMNMX clamp, MUFU
//    ex2, FFMA with W -- is interleaved into the other half's contraction, so
//    the MUFU work is spread over the FFMA2 stream instead of bursting;
//  * per-thread partials: 16-tile blocks summed in FP32, blocks accumulated in
//    FP64 (shared memory); at segment end: warp shuffles + shared memory
//    (Alg.2 l.17-20);
//  * cross-CTA: a CTA that covers a whole target tile writes V directly;
//    split tiles write fixed slots and the last arriver (one atomic counter
//    per tile, not per element) sums the slots in CTA order -- deterministic,
//    no atomics on V (replaces atomicAdd, Alg.2 l.21 P:L262).
#include "ks_internal.h"
#include "ks_ptx.cuh"

#include <cstdlib>


namespace ks {

template <int KP>
struct Fp32Cfg {
  static constexpr int kThreads = kFp32Threads;
  static constexpr int kWarps = kThreads / 32;
  static constexpr int kStages = (KP <= 8) ? 6 : 4;
  static constexpr int kRows = KP + 2;                 // coords + na + W
  static constexpr int kStageFloats = kRows * kTileS;
  static constexpr uint32_t kStageBytes = kStageFloats * 4;
  // shared layout (floats): stages | tgt [KP][256] (reused as the [2][256]
  // FP64 reduction buffer at segment end) | nb [256] | vsm double [8][512]
  // (per-thread FP64 accumulators) | mbarriers | release counters | flag
  static_assert(KP * kTileT * 4 >= 2 * kTileT * 8, "tgt must hold the FP64 reduction buffer");
  static constexpr int kTgtOff = kStages * kStageFloats;
  static constexpr int kNbOff = kTgtOff + KP * kTileT;
  static constexpr int kVsmOff = kNbOff + kTileT;            // 8-byte aligned (multiple of 128 floats)
  static constexpr int kBarOff = kVsmOff + 2 * 8 * kThreads;  // floats
  static constexpr size_t kSmemBytes = (size_t)kBarOff * 4 + kStages * 8 + kStages * 4 + 16;
};

__device__ __forceinline__ int64_t sk_start(int64_t b, int64_t U, int64_t G) { return (b * U) / G; }
// CTA that owns unit u: the largest b with floor(b*U/G) <= u.
__device__ __forceinline__ int64_t sk_owner(int64_t u, int64_t U, int64_t G) { return ((u + 1) * G - 1) / U; }

__device__ __forceinline__ uint32_t atom_add_acqrel_smem(uint32_t* p, uint32_t v) {
  uint32_t old;
  asm volatile("atom.acq_rel.cta.shared::cta.add.u32 %0, [%1], %2;"
               : "=r"(old)
               : "r"(smem_u32(p)), "r"(v)
               : "memory");
  return old;
}

// a4 + a5 for one accumulator pair: clamp (d^2 >= 0 <=> t <= 0), MUFU ex2,
// weighted accumulate into the target's pair partial sum.
__device__ __forceinline__ void epi_pair(f2_t t2, f2_t w2, float& bs) {
  float x, y, wx, wy;
  f2_unpack(t2, x, y);
  f2_unpack(w2, wx, wy);
  bs = fmaf(ex2_approx(fminf(x, 0.f)), wx, bs);
  bs = fmaf(ex2_approx(fminf(y, 0.f)), wy, bs);
}

// One half of the 8x8 micro-tile (4 targets x 8 sources = 16 pairs):
// K rank-1 FFMA2 updates (a3), with the epilogue (a4, a5) of the OTHER half's
// finished accumulators interleaved -- 16/KP pairs per k step -- so MUFU ex2
// overlaps the FFMA2 stream instead of bursting at the end of the tile.
template <int KP>
__device__ __forceinline__ void half_tile(const float* __restrict__ sp, const float* __restrict__ tg, int tx,
                                          f2_t (&acc)[4][4], const f2_t (&epi)[4][4], const f2_t (&w2)[4],
                                          float (&bs)[4]) {
#pragma unroll
  for (int k = 0; k < KP; ++k) {
    const ulonglong2 a01 = lds_pairs(sp + k * kTileS + 4 * tx);
    const ulonglong2 a23 = lds_pairs(sp + k * kTileS + 64 + 4 * tx);
    const float4 b = lds128(tg + k * kTileT);
    const f2_t av[4] = {a01.x, a01.y, a23.x, a23.y};
    const float bv[4] = {b.x, b.y, b.z, b.w};
#pragma unroll
    for (int j = 0; j < 4; ++j)
#pragma unroll
      for (int p = 0; p < 4; ++p) acc[j][p] = ffma2(f2_bcast(bv[j]), av[p], acc[j][p]);
#pragma unroll
    for (int q = 0; q < 16; ++q)
      if ((q * KP) / 16 == k) epi_pair(epi[q >> 2][q & 3], w2[q & 3], bs[q >> 2]);
  }
}

template <int KP>
__device__ __forceinline__ void init_half(const float* __restrict__ sp, const float* __restrict__ nbp, int tx,
                                          f2_t (&acc)[4][4]) {
  const ulonglong2 n01 = lds_pairs(sp + KP * kTileS + 4 * tx);
  const ulonglong2 n23 = lds_pairs(sp + KP * kTileS + 64 + 4 * tx);
  const float4 nb = lds128(nbp);
  const f2_t na[4] = {n01.x, n01.y, n23.x, n23.y};
  const float nbv[4] = {nb.x, nb.y, nb.z, nb.w};
#pragma unroll
  for (int j = 0; j < 4; ++j)
#pragma unroll
    for (int p = 0; p < 4; ++p) acc[j][p] = fadd2(f2_bcast(nbv[j]), na[p]);
}

// Full 8x8 micro-tile in one k loop (4 LDS.128 per 32 FFMA2: half the
// shared-memory traffic per FMA of the split form) with the epilogue at the
// end of the tile.
template <int KP>
__device__ __forceinline__ void full_tile(const float* __restrict__ sp, const float* __restrict__ tgt,
                                          const float* __restrict__ nbs, int tx, int ty, float (&bsA)[4],
                                          float (&bsB)[4]) {
  f2_t acc[8][4];
  {
    const ulonglong2 n01 = lds_pairs(sp + KP * kTileS + 4 * tx);
    const ulonglong2 n23 = lds_pairs(sp + KP * kTileS + 64 + 4 * tx);
    const float4 nbA = lds128(nbs + 4 * ty);
    const float4 nbB = lds128(nbs + kTileT / 2 + 4 * ty);
    const f2_t na[4] = {n01.x, n01.y, n23.x, n23.y};
    const float nb[8] = {nbA.x, nbA.y, nbA.z, nbA.w, nbB.x, nbB.y, nbB.z, nbB.w};
#pragma unroll
    for (int j = 0; j < 8; ++j)
#pragma unroll
      for (int p = 0; p < 4; ++p) acc[j][p] = fadd2(f2_bcast(nb[j]), na[p]);
  }
#pragma unroll
  for (int k = 0; k < KP; ++k) {
    const ulonglong2 a01 = lds_pairs(sp + k * kTileS + 4 * tx);
    const ulonglong2 a23 = lds_pairs(sp + k * kTileS + 64 + 4 * tx);
    const float4 bA = lds128(tgt + k * kTileT + 4 * ty);
    const float4 bB = lds128(tgt + k * kTileT + kTileT / 2 + 4 * ty);
    const f2_t av[4] = {a01.x, a01.y, a23.x, a23.y};
    const float bv[8] = {bA.x, bA.y, bA.z, bA.w, bB.x, bB.y, bB.z, bB.w};
#pragma unroll
    for (int j = 0; j < 8; ++j)
#pragma unroll
      for (int p = 0; p < 4; ++p) acc[j][p] = ffma2(f2_bcast(bv[j]), av[p], acc[j][p]);
  }
  const ulonglong2 w01 = lds_pairs(sp + (KP + 1) * kTileS + 4 * tx);
  const ulonglong2 w23 = lds_pairs(sp + (KP + 1) * kTileS + 64 + 4 * tx);
  const f2_t w2[4] = {w01.x, w01.y, w23.x, w23.y};
#pragma unroll
  for (int j = 0; j < 4; ++j)
#pragma unroll
    for (int p = 0; p < 4; ++p) {
      epi_pair(acc[j][p], w2[p], bsA[j]);
      epi_pair(acc[4 + j][p], w2[p], bsB[j]);
    }
}

template <int KP, bool SPLIT>
__global__ void __launch_bounds__(kFp32Threads, 1)
    ks_fused_fp32_kernel(const __grid_constant__ CUtensorMap tmap_src, const Fp32Args args) {
  using C = Fp32Cfg<KP>;
  constexpr int S = C::kStages;
  extern __shared__ __align__(128) float smem[];
  float* tgt = smem + C::kTgtOff;
  float* nbs = smem + C::kNbOff;
  double* vsm = reinterpret_cast<double*>(smem + C::kVsmOff);
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + C::kBarOff);
  uint32_t* relcnt = reinterpret_cast<uint32_t*>(full + S);
  int* flag = reinterpret_cast<int*>(relcnt + S);

  const int tid = threadIdx.x;
  const int warp = tid >> 5, lane = tid & 31;
  // lane bits: b0 -> tx bit 0, b1..b2 -> ty, b3..b4 -> tx bits 1..2.  Each
  // quarter-warp (8 lanes) then touches 2 source chunks and 4 target chunks,
  // so an LDS.128 is served in 2 shared-memory wavefronts instead of 4.
  const int tx = (warp & 1) * 8 + ((lane & 1) | ((lane >> 2) & 6));  // source micro-column 0..15
  const int ty = (warp >> 1) * 4 + ((lane >> 1) & 3);               // target micro-row 0..31
  // this thread: sources {4tx..4tx+3} U {64+4tx..}, targets A = {4ty..4ty+3}, B = {128+4ty..}

  const int64_t U = args.sk.units, G = args.sk.grid;
  const int n_s = args.sk.n_s;
  const int64_t b = blockIdx.x;
  const int64_t u_begin = sk_start(b, U, G), u_end = sk_start(b + 1, U, G);
  const int count = (int)(u_end - u_begin);

  if (args.cta_times != nullptr && tid == 0) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    args.cta_times[2 * b] = t;
  }
  if (tid == 0) {
    tma_prefetch_desc(&tmap_src);
    for (int s = 0; s < S; ++s) {
      mbar_init(&full[s], 1);
      relcnt[s] = 0;
    }
    fence_mbar_init();
  }
  __syncthreads();
  if (tid == 0) {
    for (int s = 0; s < S && s < count; ++s) {
      const int64_t u = u_begin + s;
      mbar_arrive_expect_tx(&full[s], C::kStageBytes);
      tma_load_2d(smem + s * C::kStageFloats, &tmap_src, (int32_t)((u % n_s) * kTileS), 0, &full[s]);
    }
  }

  const double c = args.c;
  int q = 0;  // local unit index
  int64_t u = u_begin;
  while (u < u_end) {
    const int64_t tt = u / n_s;
    const int st0 = (int)(u % n_s);
    const int seg = (int)((u_end - u < (int64_t)(n_s - st0)) ? (u_end - u) : (int64_t)(n_s - st0));

    // ---------------- a2: target prologue (centre, norm, stage in smem)
    __syncthreads();  // previous segment finished with tgt / nbs
    {
      const int j = tid >> 1, half = tid & 1;
      const int64_t row = tt * kTileT + j;
      const bool live = row < args.N;
      const float* bp = args.beta + row * args.K;
      double n = 0.0;
#pragma unroll
      for (int dd = 0; dd < KP / 2; ++dd) {
        const int d = half * (KP / 2) + dd;
        float x = 0.f;
        if (live && d < args.K) x = __ldg(bp + d) - __ldg(args.mu + d);
        n += (double)x * (double)x;
        tgt[d * kTileT + j] = x;
      }
      n += __shfl_xor_sync(0xffffffffu, n, 1);
      if (half == 0) nbs[j] = (float)(-c * n);
    }
#pragma unroll
    for (int j = 0; j < 8; ++j) vsm[j * C::kThreads + tid] = 0.0;
    __syncthreads();

    float bsA[4], bsB[4];      // per-target FP32 partial sums (<= 16 tiles)
    f2_t accA[4][4], accB[4][4];
    f2_t w2[4];
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      bsA[j] = 0.f;
      bsB[j] = 0.f;
#pragma unroll
      for (int p = 0; p < 4; ++p) accB[j][p] = f2_bcast(-INFINITY);  // "pending" epilogue adds ex2(-inf) = 0
    }
#pragma unroll
    for (int p = 0; p < 4; ++p) w2[p] = f2_bcast(0.f);

    for (int e = 0; e < seg; ++e, ++q) {
      const int s = q % S;
      const uint32_t ph = (uint32_t)((q / S) & 1);
      mbar_wait(&full[s], ph);
      const float* sp = smem + s * C::kStageFloats;

      if constexpr (!SPLIT) {
        full_tile<KP>(sp, tgt, nbs, tx, ty, bsA, bsB);
      } else {
      // targets A: contraction; epilogue of the previous tile's half B
      init_half<KP>(sp, nbs + 4 * ty, tx, accA);
      half_tile<KP>(sp, tgt + 4 * ty, tx, accA, accB, w2, bsB);
      {
        const ulonglong2 w01 = lds_pairs(sp + (KP + 1) * kTileS + 4 * tx);
        const ulonglong2 w23 = lds_pairs(sp + (KP + 1) * kTileS + 64 + 4 * tx);
        w2[0] = w01.x; w2[1] = w01.y; w2[2] = w23.x; w2[3] = w23.y;
      }
      // targets B: contraction; epilogue of this tile's half A
      __syncwarp();
      init_half<KP>(sp, nbs + kTileT / 2 + 4 * ty, tx, accB);
      half_tile<KP>(sp, tgt + kTileT / 2 + 4 * ty, tx, accB, accA, w2, bsA);
      }

      // release the stage; the last warp to release it refills it (unit q + S)
      __syncwarp();
      if (lane == 0) {
        const uint32_t old = atom_add_acqrel_smem(&relcnt[s], 1u);
        if (old == (uint32_t)(C::kWarps - 1)) {
          relcnt[s] = 0u;
          if (q + S < count) {
            const int64_t un = u_begin + q + S;
            fence_proxy_async_smem();
            mbar_arrive_expect_tx(&full[s], C::kStageBytes);
            tma_load_2d(smem + s * C::kStageFloats, &tmap_src, (int32_t)((un % n_s) * kTileS), 0, &full[s]);
          }
        }
      }
      if ((e & 15) == 15) {
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          vsm[j * C::kThreads + tid] += (double)bsA[j];
          vsm[(4 + j) * C::kThreads + tid] += (double)bsB[j];
          bsA[j] = 0.f;
          bsB[j] = 0.f;
        }
      }
    }
    // drain: epilogue of the last tile's half B
    if constexpr (SPLIT) {
#pragma unroll
      for (int qq = 0; qq < 16; ++qq) epi_pair(accB[qq >> 2][qq & 3], w2[qq & 3], bsB[qq >> 2]);
    }
    double vacc[8];
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      vacc[j] = vsm[j * C::kThreads + tid] + (double)bsA[j];
      vacc[4 + j] = vsm[(4 + j) * C::kThreads + tid] + (double)bsB[j];
    }

    // ---------------- a5: reduce the 16 source micro-columns of each target
    // lanes with equal ty share targets: xor over the tx lane bits 0, 3, 4
#pragma unroll
    for (int jj = 0; jj < 8; ++jj) {
      double v = vacc[jj];
      v += __shfl_xor_sync(0xffffffffu, v, 1);
      v += __shfl_xor_sync(0xffffffffu, v, 8);
      v += __shfl_xor_sync(0xffffffffu, v, 16);
      vacc[jj] = v;
    }
    // warps 2m and 2m+1 share targets: combine through smem in fixed order
    double* redd = reinterpret_cast<double*>(tgt);  // tgt is free after the last tile
    __syncthreads();
    if ((lane & 0x19) == 0) {  // tx lane bits zero: one writer per ty
#pragma unroll
      for (int jj = 0; jj < 8; ++jj) {
        const int j = (jj < 4) ? (4 * ty + jj) : (kTileT / 2 + 4 * ty + jj - 4);
        redd[(warp & 1) * kTileT + j] = vacc[jj];
      }
    }
    __syncthreads();

    // ---------------- a6 + a7: write V, or a partial + deterministic fix-up
    const bool whole = (st0 == 0) && (seg == n_s);
    if (whole) {
      if (tid < kTileT) {
        const int64_t row = tt * kTileT + tid;
        if (row < args.N) args.V[row] = (float)(redd[tid] + redd[kTileT + tid]);
      }
    } else {
      const int first_tile_of_b = (int)(u_begin / n_s);
      const int slot = (tt == first_tile_of_b) ? 0 : 1;
      if (tid < kTileT) {
        args.partial[(b * 2 + slot) * kTileT + tid] = (float)(redd[tid] + redd[kTileT + tid]);
        __threadfence();
      }
      __syncthreads();
      const int64_t b_first = sk_owner(tt * n_s, U, G);
      const int64_t b_last = sk_owner(tt * n_s + n_s - 1, U, G);
      if (tid == 0) {
        const int old = atomicAdd(&args.counters[tt], 1);
        const int last = (old == (int)(b_last - b_first));
        if (last) args.counters[tt] = 0;  // leave zero for the next launch
        *flag = last;
      }
      __syncthreads();
      if (*flag && tid < kTileT) {
        __threadfence();
        float sum = 0.f;
        for (int64_t bb = b_first; bb <= b_last; ++bb) {
          const int sl = (tt == sk_start(bb, U, G) / n_s) ? 0 : 1;
          sum += __ldcg(&args.partial[(bb * 2 + sl) * kTileT + tid]);
        }
        const int64_t row = tt * kTileT + tid;
        if (row < args.N) args.V[row] = sum;
      }
    }
    u += seg;
  }
  if (args.cta_times != nullptr && tid == 0) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    args.cta_times[2 * b + 1] = t;
  }
}

// Tile-body variant.  Measured on B200 (SS7): at K = 32 the split
// halves with the interleaved epilogue are faster (76% vs 74% of the FP32
// roofline); at K <= 16 the full 8x8 tile (half the LDS per FMA) wins.
// KS_OPT_FP32_SPLIT=0/1 overrides (tuning option).
template <int KP>
static bool fp32_split() {
  const int o = opt(KS_OPT_FP32_SPLIT, -1);
  return (o == 0 || o == 1) ? o == 1 : KP >= 32;
}

template <int KP, bool SPLIT>
static cudaError_t launch_kps(const CUtensorMap* tmap, const Fp32Args& a, cudaStream_t st) {
  using C = Fp32Cfg<KP>;
  static std::atomic<uint64_t> attr_done{0};
  cudaError_t e = smem_optin_once(attr_done, reinterpret_cast<const void*>(ks_fused_fp32_kernel<KP, SPLIT>),
                                  (int)C::kSmemBytes);
  if (e != cudaSuccess) return e;
  ks_fused_fp32_kernel<KP, SPLIT><<<a.sk.grid, C::kThreads, C::kSmemBytes, st>>>(*tmap, a);
  return cudaGetLastError();
}

template <int KP>
static cudaError_t launch_kp(const CUtensorMap* tmap, const Fp32Args& a, cudaStream_t st) {
  return fp32_split<KP>() ? launch_kps<KP, true>(tmap, a, st) : launch_kps<KP, false>(tmap, a, st);
}

cudaError_t launch_fused_fp32(const CUtensorMap* tmap_src, int k_pad, const Fp32Args& a, cudaStream_t st) {
  switch (k_pad) {
    case 4: return launch_kp<4>(tmap_src, a, st);
    case 8: return launch_kp<8>(tmap_src, a, st);
    case 16: return launch_kp<16>(tmap_src, a, st);
    case 32: return launch_kp<32>(tmap_src, a, st);
    default: return cudaErrorInvalidValue;
  }
}

template <int KP>
static int ctas_per_sm_kp() {
  using C = Fp32Cfg<KP>;
  int n = 0;
  cudaFuncSetAttribute(ks_fused_fp32_kernel<KP, false>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                       (int)C::kSmemBytes);
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, ks_fused_fp32_kernel<KP, false>, C::kThreads,
                                                    C::kSmemBytes) != cudaSuccess)
    n = 1;
  return n < 1 ? 1 : n;
}

int fused_fp32_ctas_per_sm(int k_pad) {
  switch (k_pad) {
    case 4: return ctas_per_sm_kp<4>();
    case 8: return ctas_per_sm_kp<8>();
    case 16: return ctas_per_sm_kp<16>();
    default: return ctas_per_sm_kp<32>();
  }
}

int fused_fp32_stages(int k_pad) {
  switch (k_pad) {
    case 4: return Fp32Cfg<4>::kStages;
    case 8: return Fp32Cfg<8>::kStages;
    case 16: return Fp32Cfg<16>::kStages;
    default: return Fp32Cfg<32>::kStages;
  }
}

}  // namespace ks
