// ks_fused_rv.cu -- the fused tensor-core kernel for several weight columns (R > 1, split-FP16,
// K + 6 <= 64): the weighted sum runs as a second tcgen05 contraction on the R = 1 kernel's
// skeleton (scope rows a2-a7; R columns are the north_star extension of Eq.2).
//
// What it computes (PAPER.md SS III-C, Alg.2; Eq.1-3):
//   t_ji = sum_d bh_jd a_id + na_i + nb_j = -c d_ji^2  (one accumulator: split-FP16 coordinates
//                                              and the folded norm pieces, readings Q26 / Q28)
//   P_ji = 2^-|t_ji|                          (|d^2|: the d^2 >= 0 clamp up to the rounding of
//                                              d^2, reading Q8; MUFU.EX2, part on the FMA pipe)
//   V_jr = sum_i P_ji W_ir                    (Eq.2, per weight column)
// P is split into FP16 hi/lo and written back over its own S columns, W as FP16 hi/lo of
// per-column power-of-2 scaled weights, and V = P_hi [W_hi | W_lo] + P_lo W_hi accumulates in
// TMEM (reading Q27), folded into compensated FP32 row sums and unscaled by 2^-s_r.
//
// Structure: one persistent 672-thread CTA per SM over (128-target x 96-source) units, the
// same wave + stream-K schedule and deterministic fix-up as ks_fused_r1.cu:
//   warp 0    TMA producer: target planes once per target tile (two buffers), each unit's
//             source planes into a D-stage ring;
//   warps 1,3 S-MMA issuers (even / odd units) into TMEM S buffer q % 4;
//   warp 2    TMEM allocation; the V-MMA issuer (unit order: one issuer, so the TMEM
//             accumulation order is fixed -> bitwise deterministic);
//   warp 20   TMA producer of each unit's weight tile ([W_hi | W_lo] rows, 96 sources);
//   warps 4..19  4 epilogue groups of 4 warps, one per TMEM lane quarter (group q % 4 computes
//             unit q's P in S buffer q % 4 and writes it back in place, then releases it to the
//             V issuer; the V issuer releases the buffer to the next S MMA as soon as it has
//             *issued* the unit's V MMAs -- tcgen05.mma ops execute in issue order); every
//             epilogue warp also folds RC / 4 columns of each V block (<= kRvBlock units of a
//             target tile) from TMEM into compensated FP32 shared-memory row sums and, at a
//             target tile's end, writes them to V or a stream-K partial.  (Two groups of 8
//             warps, each alternating between two buffers, measured 2% slower: a group's next S
//             waited on the other buffer's V.)
// Units are 128 targets x 96 sources.  TMEM: 4 S buffers x 96 columns | 2 V blocks x 2 RC columns
// (RC = 16: [V_hh+lh | V_hl]; RC = 32: the two 16-column groups side by side).
#include "ks_internal.h"
#include <cuda_fp16.h>
#include "ks_ptx.cuh"

#ifndef KS_DEBUG
#define KS_DEBUG 0
#endif

// KS_DEBUG builds: every wait is bounded; a wait that spins ~10^8 times prints where it hangs and traps
#if KS_DEBUG
#include <cstdio>
#define RV_WAIT(bar, par, tag, qv)                                                                           \
  do {                                                                                                       \
    long long spins_ = 0;                                                                                    \
    while (!mbar_try_wait(smem_u32(bar), (par))) {                                                           \
      ++spins_;                                                                                              \
      if (spins_ == (1ll << 21) && (threadIdx.x & 31) == 0)                                                  \
        printf("rv hang: cta %d warp %d at %s q=%d par=%u\n", (int)blockIdx.x, (int)(threadIdx.x >> 5), tag,  \
               (int)(qv), (unsigned)(par));                                                                  \
      if (spins_ == (1ll << 23)) __trap();                                                                   \
    }                                                                                                        \
  } while (0)
#else
#define RV_WAIT(bar, par, tag, qv) mbar_wait((bar), (par))
#endif

#ifndef KS_TRACE
#define KS_TRACE 0
#endif
#if KS_TRACE
// CTA 0, per unit: S MMAs issued, epilogue S ready, P ready, V MMAs issued (clock64)
#define RV_TRACE(q, k) \
  if (args.trace != nullptr && blockIdx.x == 0 && (q) < 4096) args.trace[12 * (q) + (k)] = (unsigned long long)clock64()
#else
#define RV_TRACE(q, k) (void)0
#endif

namespace ks {

namespace {

constexpr int kRvEpiWarps = 16;
constexpr int kRvThreads = 128 + 32 * kRvEpiWarps + 32;  // + the weight producer (warp 20)
constexpr int kRvSBufs = 4;          // S buffers (TMEM columns 0..383)
constexpr int kRvTS = kRvTileS;            // sources per unit (4 x 96 S columns + 2 V blocks fit 512)
constexpr uint32_t kRvPlane = 128u * 64u;   // target plane (128 rows x 64 B); source planes 96 rows
constexpr int kRvMaxStages = 8;
constexpr int kRvBlock = 8;          // units per V block (FP32 TMEM accumulation over <= 768 sources;
                                     // 4 measured 2% slower: the V issuer waits for all 16 warps'
                                     // fold of the block two back)
constexpr uint32_t kRvSmem = 227u * 1024u;
constexpr uint32_t kRvBars = 1024u;
constexpr uint32_t kRvColV = kRvSBufs * kRvTS;  // 384

__device__ __forceinline__ int64_t rv_sk_start(int64_t b, int64_t U, int64_t G) { return (b * U) / G; }
__device__ __forceinline__ int64_t rv_sk_owner(int64_t u, int64_t U, int64_t G) { return ((u + 1) * G - 1) / U; }

struct RvSched {
  int64_t G, b, waves, rem_t0, Urem, Gr, v0;
  int n_s, qw, count;
  __device__ void init(int64_t n_t, int ns, int64_t grid, int64_t blk) {
    n_s = ns;
    G = grid;
    b = blk;
    waves = n_t / G;
    rem_t0 = waves * G;
    Urem = (n_t - rem_t0) * n_s;
    Gr = Urem < G ? Urem : G;
    qw = (int)(waves * n_s);
    int64_t v1 = 0;
    v0 = 0;
    if (b < Gr) {
      v0 = rv_sk_start(b, Urem, Gr);
      v1 = rv_sk_start(b + 1, Urem, Gr);
    }
    count = qw + (int)(v1 - v0);
  }
  // the segment (run of one target tile's units) starting at local unit q
  __device__ void segment(int q, int64_t& tt, int& st0, int& len) const {
    if (q < qw) {
      tt = b + (int64_t)(q / n_s) * G;
      st0 = 0;
      len = n_s;
    } else {
      const int64_t v = v0 + (q - qw);
      tt = rem_t0 + v / n_s;
      st0 = (int)(v % n_s);
      len = n_s - st0 < count - q ? n_s - st0 : count - q;
    }
  }
};

// kind::f16 MMA with A (P, FP16 pairs) in TMEM and B from a shared-memory descriptor given as its
// low word + shared high word (uniform-datapath issue, like mma_f16_lo).
__device__ __forceinline__ void mma_f16_ts_lo(uint32_t d_tmem, uint32_t a_tmem, uint32_t b_lo, uint32_t desc_hi,
                                              uint32_t idesc, uint32_t accumulate, uint32_t issue) {
  asm volatile(
      "{\n\t.reg .pred p, q;\n\t.reg .b64 db;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "setp.ne.b32 q, %6, 0;\n\t"
      "mov.b64 db, {%2, %5};\n\t"
      "@q tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], db, %3, p;\n\t}" ::"r"(d_tmem),
      "r"(a_tmem), "r"(b_lo), "r"(idesc), "r"(accumulate), "r"(desc_hi), "r"(issue)
      : "memory");
}

// f32x2 subtract (one FMA-pipe issue for a pair)
__device__ __forceinline__ f2_t fsub2(f2_t a, f2_t b) {
  f2_t d;
  asm("sub.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(a), "l"(b));
  return d;
}

// One NC-column batch of P for a lane: P = 2^-|t| (t = -c d^2 from the MMA; the reflection |d^2|
// keeps P <= exp(0) = 1 -- the d^2 >= 0 clamp up to the rounding of d^2, reading Q8 -- and costs
// nothing: MUFU.EX2 takes -|x| as an operand modifier), NPOLY of every 16 pairs on the FMA pipe;
// split P = hi + lo in FP16 (hi = P with its low 13 mantissa bits cleared, exact for P >= 2^-14;
// lo the remainder, one f32x2 subtract per pair), packed in place: words 0-7 hi pairs and 8-15
// lo pairs of sources 0-15, 16-23 / 24-31 of sources 16-31 (one 16-source K step of the V MMA
// each).  P below 2^-14 is an FP16 subnormal: absolute error <= 2^-25 per term, <= 2^-25 sum |W|
// in V (reading Q27).
template <int NPOLY, int NC>
__device__ __forceinline__ void rv_batch(uint32_t (&sv)[NC]) {
  uint32_t out[NC];
#pragma unroll
  for (int k = 0; k < NC / 2; ++k) {  // pair k = sources (2k, 2k + 1)
    const float t0 = -fabsf(__uint_as_float(sv[2 * k])), t1 = -fabsf(__uint_as_float(sv[2 * k + 1]));
    float p0, p1;
    if (((k * NPOLY) & 15) < NPOLY) {
      f2_unpack(exp2_poly2(f2_pack(fmaxf(t0, -125.f), fmaxf(t1, -125.f))), p0, p1);
    } else {
      p0 = ex2_approx(t0);
      p1 = ex2_approx(t1);
    }
    const float h0 = __uint_as_float(__float_as_uint(p0) & 0xFFFFE000u);
    const float h1 = __uint_as_float(__float_as_uint(p1) & 0xFFFFE000u);
    const __half2 hv = __floats2half2_rn(h0, h1);
    float l0, l1;
    f2_unpack(fsub2(f2_pack(p0, p1), f2_pack(h0, h1)), l0, l1);
    const __half2 lv = __floats2half2_rn(l0, l1);
    const int step = k >> 3, w = k & 7;
    out[16 * step + w] = *reinterpret_cast<const uint32_t*>(&hv);
    out[16 * step + 8 + w] = *reinterpret_cast<const uint32_t*>(&lv);
  }
#pragma unroll
  for (int i = 0; i < NC; ++i) sv[i] = out[i];
}

__device__ __forceinline__ int rv_wcol_exp(unsigned bits) {
  const float m = __uint_as_float(bits);
  if (!(m > 0.f) || !(m <= 3.0e38f)) return 0;
  int e;
  frexpf(m, &e);
  return 15 - e;
}

}  // namespace

template <int NPOLY, int RC>
__global__ void __launch_bounds__(kRvThreads, 1)
    ks_fused_rv_kernel(const __grid_constant__ CUtensorMap mA_hi, const __grid_constant__ CUtensorMap mA_lo,
                       const __grid_constant__ CUtensorMap mB_hi, const __grid_constant__ CUtensorMap mB_lo,
                       const __grid_constant__ CUtensorMap mW, const RvArgs args) {
  extern __shared__ __align__(1024) uint8_t smem[];
  if ((smem_u32(smem) & 1023u) != 0u) __trap();
  const int tid = threadIdx.x, warp = __shfl_sync(0xffffffffu, tid >> 5, 0), lane = tid & 31;
  const int64_t b = blockIdx.x;
  if (args.cta_times != nullptr && threadIdx.x == 0) {  // KS_OPT_MEASURE_CLOCK: effective SM clock
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    args.cta_times[4 * b] = t;
    args.cta_times[4 * b + 1] = (unsigned long long)clock64();
  }
  constexpr uint32_t kWSlot = (uint32_t)RC * 2u * kRvTS * 2u;  // [W_hi | W_lo] rows x 96 sources (FP16)
  // weight ring depth: a slot is refilled only after the V MMA of the unit kRvWSlots back has
  // completed, so the ring must cover that latency plus a TMA round trip (measured: 4 slots left
  // the V issuer waiting ~700 cycles per unit on weights at RC = 16)
  constexpr int kRvWSlots = RC == 16 ? 8 : 4;
  constexpr uint32_t kVAcc = 128u * RC * 8u;                   // row sums + compensations (FP32)

  // ---- geometry
  const int n_kc = args.n_kc;
  const bool narrow = args.narrow != 0;
  const bool lo1 = n_kc == 2 && args.kdims > 32;
  const int P = 2 + (n_kc == 2 ? (lo1 ? 2 : 1) : 0);
  const uint32_t plane = narrow ? kRvPlane / 2 : kRvPlane;  // target (A) plane
  const uint32_t planeB = plane / 128u * kRvTS;               // source (B) plane
  const uint32_t tile_bytes = (uint32_t)P * plane, tileB = (uint32_t)P * planeB;
  const uint32_t region = kRvSmem - kRvBars - kVAcc - kRvWSlots * kWSlot;
  int D = (int)((region - 2 * tile_bytes) / tileB);
  if (D > kRvMaxStages) D = kRvMaxStages;
  D &= ~1;  // even: units q and q + D then come from the same S-MMA warp, which therefore waits on
            // every phase of a stage barrier (a parity wait must never skip a phase)
  const uint32_t offA = 0, offS = 2 * tile_bytes;
  uint8_t* wring = smem + region;
  // compensated FP32 row accumulators [sum | compensation][RC][128] (lane-consecutive rows)
  float* vacc = reinterpret_cast<float*>(smem + region + kRvWSlots * kWSlot);
  float* vcmp = vacc + RC * 128;
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem + kRvSmem - kRvBars);
  uint64_t* full = bars;                      // [8]
  uint64_t* empty = full + kRvMaxStages;      // [8]
  uint64_t* afull = empty + kRvMaxStages;     // [2]
  uint64_t* aempty = afull + 2;               // [2]
  // Phase bookkeeping: an mbarrier parity wait must never be more than one phase behind, so a
  // barrier is only shared by units its waiter waits for consecutively: S buffer q % 4 is filled
  // by warp 1 / 3 (q & 1), read by group q % 2 and released by the V issuer, so every waiter
  // of sfull / sempty / pready[q % 4] waits on each of its phases.
  uint64_t* sfull = aempty + 2;               // [4]
  uint64_t* sempty = sfull + kRvSBufs;        // [4]
  uint64_t* pready = sempty + kRvSBufs;       // [4]
  uint64_t* wfull = pready + kRvSBufs;        // [kRvWSlots]
  uint64_t* wempty = wfull + kRvWSlots;       // [kRvWSlots]
  uint64_t* vfull = wempty + kRvWSlots;       // [2]
  uint64_t* vempty = vfull + 2;               // [2]
  uint32_t* tmem_base_smem = reinterpret_cast<uint32_t*>(vempty + 2);
  int* flag = reinterpret_cast<int*>(tmem_base_smem + 1);

  RvSched sc;
  sc.init(args.sk.n_t, args.sk.n_s, args.sk.grid, b);
  const int count = sc.count;
  const int n_s = sc.n_s;

  if (tid == 0) {
    for (int i = 0; i < kRvMaxStages; ++i) {
      mbar_init(&full[i], 1);
      mbar_init(&empty[i], 1);
    }
    for (int i = 0; i < 2; ++i) {
      mbar_init(&afull[i], 1);
      mbar_init(&aempty[i], 2);  // both S-MMA warps
      mbar_init(&vfull[i], 1);
      mbar_init(&vempty[i], kRvEpiWarps);  // every epilogue warp folds a share of each block
    }
    for (int i = 0; i < kRvSBufs; ++i) {
      mbar_init(&sfull[i], 1);
      mbar_init(&sempty[i], 1);
      mbar_init(&pready[i], 4);  // the unit's group (4 warps)
    }
    for (int i = 0; i < kRvWSlots; ++i) {
      mbar_init(&wfull[i], 1);
      mbar_init(&wempty[i], 1);
    }
    fence_mbar_init();
  }
  if (warp == 2) tmem_alloc(tmem_base_smem, 512);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tbase = __shfl_sync(0xffffffffu, *tmem_base_smem, 0);
  pdl_wait();

  if (warp == 0) {
    // ================= TMA producer of the target and source operand planes
    const bool leader = elect_one();
    if (leader) {
      tma_prefetch_desc(&mA_hi);
      tma_prefetch_desc(&mB_hi);
    }
    int s = 0;
    uint32_t ph = 0;
    int seg = -1;
    for (int q = 0; q < count;) {
      int64_t tt;
      int st0, len;
      sc.segment(q, tt, st0, len);
      ++seg;
      const int ab = seg & 1;
      RV_WAIT(&aempty[ab], (uint32_t)(((seg >> 1) & 1) ^ 1), "aempty", seg);
      if (leader) {
        uint8_t* ap = smem + offA + ab * tile_bytes;
        const int y = (int)(tt * 128);
        mbar_arrive_expect_tx(&afull[ab], tile_bytes);
        tma_load_2d(ap, &mA_hi, 0, y, &afull[ab]);
        tma_load_2d(ap + plane, &mA_lo, 0, y, &afull[ab]);
        if (n_kc == 2) {
          tma_load_2d(ap + 2 * plane, &mA_hi, 32, y, &afull[ab]);
          if (lo1) tma_load_2d(ap + 3 * plane, &mA_lo, 32, y, &afull[ab]);
        }
      }
      __syncwarp();
      for (int j = 0; j < len; ++j, ++q) {
        RV_WAIT(&empty[s], ph ^ 1u, "empty", q);
        if (leader) {
          uint8_t* sp = smem + offS + s * tileB;
          const int y = (st0 + j) * kRvTS;
          mbar_arrive_expect_tx(&full[s], tileB);
          tma_load_2d(sp, &mB_hi, 0, y, &full[s]);
          tma_load_2d(sp + planeB, &mB_lo, 0, y, &full[s]);
          if (n_kc == 2) {
            tma_load_2d(sp + 2 * planeB, &mB_hi, 32, y, &full[s]);
            if (lo1) tma_load_2d(sp + 3 * planeB, &mB_lo, 32, y, &full[s]);
          }
        }
        __syncwarp();
        if (++s == D) {
          s = 0;
          ph ^= 1u;
        }
      }
    }
  } else if (warp == 20) {
    // ================= TMA producer of the weight tiles (one [W_hi | W_lo] box per unit)
    const bool leader = elect_one();
    if (leader) tma_prefetch_desc(&mW);
    int q = 0;
    for (int q0 = 0; q0 < count;) {
      int64_t tt;
      int st0, len;
      sc.segment(q0, tt, st0, len);
      for (int j = 0; j < len; ++j, ++q) {
        const int slot = q % kRvWSlots;
        RV_WAIT(&wempty[slot], (uint32_t)(((q / kRvWSlots) & 1) ^ 1), "wempty", q);
        if (leader) {
          mbar_arrive_expect_tx(&wfull[slot], kWSlot);
          tma_load_3d(wring + slot * kWSlot, &mW, 0, 2 * args.r_off, (st0 + j) * (kRvTS / 32), &wfull[slot]);
        }
        __syncwarp();
      }
      q0 += len;
    }
  } else if (warp == 1 || warp == 3) {
    // ================= S-MMA issuers (even / odd units), uniform datapath (as ks_fused_r1.cu)
    const int mine = warp == 1 ? 0 : 1;
    const uint32_t lead = elect_one() ? 1u : 0u;
    const uint32_t idS = idesc_f16(128, kRvTS);
    uint32_t plan = 0;
    for (int st4 = 0; st4 < (narrow ? 1 : 2 * n_kc); ++st4) {
      const int col0 = st4 * 16;
      const uint32_t np = col0 >= args.kcols ? 0u : (col0 >= args.kdims ? 1u : 3u);
      plan |= np << (2 * st4);
    }
    const uint32_t dhi = (uint32_t)((narrow ? sdesc_k_sw32(smem) : sdesc_k_sw64(smem)) >> 32);
    const uint32_t dA0 = (uint32_t)sdesc_k_sw64(smem + offA), dS0 = (uint32_t)sdesc_k_sw64(smem + offS);
    const uint32_t kP16 = plane >> 4, kPB16 = planeB >> 4;
    const uint32_t tile16 = tile_bytes >> 4, tileB16 = tileB >> 4;
    int s = 0, bq = 0, u3 = 0;  // stage; S buffer q % 4 and its use count q / 4
    uint32_t ph = 0;
    int seg = -1;
    int q = 0;
    for (int q0 = 0; q0 < count;) {
      int64_t tt;
      int st0, len;
      sc.segment(q0, tt, st0, len);
      if (seg >= 0) tc_commit_if(&aempty[seg & 1], lead);
      ++seg;
      RV_WAIT(&afull[seg & 1], (uint32_t)((seg >> 1) & 1), "afull", seg);
      for (int j = 0; j < len; ++j, ++q) {
        if ((q & 1) == mine) {
          if (u3 > 0) RV_WAIT(&sempty[bq], (uint32_t)((u3 - 1) & 1), "sempty", q);  // V MMA of unit q - 4 done
          RV_WAIT(&full[s], ph, "full", q);
          if (lane == 0) RV_TRACE(q, 4);
          tc_fence_after();
          const uint32_t dS = tbase + (uint32_t)(bq * kRvTS);
          const uint32_t aT = dA0 + (uint32_t)(seg & 1) * tile16, bT = dS0 + (uint32_t)s * tileB16;
#pragma unroll
          for (int kc = 0; kc < 2; ++kc) {
            if (kc >= n_kc) break;
            const uint32_t pl = kc == 0 ? 0u : 2u;
            const uint32_t aH = aT + pl * kP16, aL = aH + kP16, bH = bT + pl * kPB16, bL = bH + kPB16;
#pragma unroll
            for (int ks = 0; ks < 2; ++ks) {
              const uint32_t np = (plan >> (2 * (2 * kc + ks))) & 3u;
              const uint32_t o = (uint32_t)(ks * 2);
              const uint32_t acc0 = (kc > 0 || ks > 0) ? 1u : 0u;
              if (KS_DEBUG && (args.dbg & 2)) continue;
              if (np == 3u) {
                mma_f16_lo(dS, aL + o, bH + o, dhi, idS, acc0, lead);
                mma_f16_lo(dS, aH + o, bL + o, dhi, idS, 1u, lead);
                mma_f16_lo(dS, aH + o, bH + o, dhi, idS, 1u, lead);
              } else if (np == 1u) {
                mma_f16_lo(dS, aH + o, bH + o, dhi, idS, acc0, lead);
              }
            }
          }
          tc_commit_if(&empty[s], lead);
          tc_commit_if(&sfull[bq], lead);
          if (lane == 0) RV_TRACE(q, 0);
        }
        if (++s == D) {
          s = 0;
          ph ^= 1u;
        }
        if (++bq == kRvSBufs) {
          bq = 0;
          ++u3;
        }
      }
      q0 += len;
    }
  } else if (warp == 2) {
    // ================= V-MMA issuer, units in order (deterministic accumulation order)
    const uint32_t lead = elect_one() ? 1u : 0u;
    const uint32_t idV2 = idesc_f16(128, 2 * RC), idV1 = idesc_f16(128, 16);
    const uint32_t whi = (uint32_t)(sdesc_k_sw64(smem) >> 32);
    const uint32_t w0 = (uint32_t)sdesc_k_sw64(wring);
    int bq = 0, u3 = 0, blk = 0;
    int q = 0;
    for (int q0 = 0; q0 < count;) {
      int64_t tt;
      int st0, len;
      sc.segment(q0, tt, st0, len);
      for (int j = 0; j < len; ++j, ++q) {
        const int jb = j % kRvBlock;
        const bool first = jb == 0, last = jb == kRvBlock - 1 || j == len - 1;
        const int slot = q % kRvWSlots;
        if (first && blk >= 2) RV_WAIT(&vempty[blk & 1], (uint32_t)(((blk >> 1) - 1) & 1), "vempty", blk);
        if (lane == 0) RV_TRACE(q, 6);
        RV_WAIT(&pready[bq], (uint32_t)(u3 & 1), "pready", q);
        if (lane == 0) RV_TRACE(q, 7);
        RV_WAIT(&wfull[slot], (uint32_t)((q / kRvWSlots) & 1), "wfull", q);
        if (lane == 0) RV_TRACE(q, 5);
        tc_fence_after();
        const uint32_t dV = tbase + kRvColV + (uint32_t)((blk & 1) * 2 * RC);
        const uint32_t aP = tbase + (uint32_t)(bq * kRvTS);
        const uint32_t wb = w0 + (uint32_t)((slot * kWSlot) >> 4);
#pragma unroll
        for (int kk = 0; kk < kRvTS / 16; ++kk) {  // 16 sources per K step
          if (KS_DEBUG && (args.dbg & 1)) break;
          const uint32_t bd = wb + (uint32_t)((((kk >> 1) * (2 * RC * 64)) + (kk & 1) * 32) >> 4);
          const uint32_t aHi = aP + 16u * kk;
          mma_f16_ts_lo(dV, aHi, bd, whi, idV2, (first && kk == 0) ? 0u : 1u, lead);
#pragma unroll
          for (int g = 0; g < RC / 16; ++g)
            mma_f16_ts_lo(dV + 32u * g, aHi + 8u, bd + (uint32_t)((g * 32 * 64) >> 4), whi, idV1, 1u, lead);
        }
        // the S buffer may take unit q + 4's S MMAs as soon as this unit's V MMAs are *issued*:
        // tcgen05.mma ops execute in issue order, so the V MMAs read P before the next S MMA
        // overwrites it (a commit here would add the V execution and the commit round trip to
        // every group's wait for its next unit)
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(&sempty[bq]);
        tc_commit_if(&wempty[slot], lead);
        if (lane == 0) RV_TRACE(q, 3);
        if (last) {
          tc_commit_if(&vfull[blk & 1], lead);
          ++blk;
        }
        if (++bq == kRvSBufs) {
          bq = 0;
          ++u3;
        }
      }
      q0 += len;
    }
  } else if (warp >= 4 && warp < 20) {
    // ================= epilogue: group gr (4 warps, one per TMEM lane quarter g) computes P of the
    // units q % 4 == gr in S buffer gr; every warp also folds RC / 4 weight columns of V (the
    // fold's work and latency split over all 16 warps)
    const int ew = warp - 4;
    const int g = ew & 3, gr = ew >> 2;      // TMEM lane quarter, group (= S buffer, units q % 4 == gr)
    constexpr int kNC = RC / 4;              // weight columns this warp folds
    const int rlo = gr * kNC;                // first of them
    const int rhi = rlo + kNC;
    const int row = 32 * g + lane;
    const uint32_t lane_off = (uint32_t)(32 * g) << 16;
    for (int r = rlo; r < rhi; ++r) vacc[r * 128 + row] = vcmp[r * 128 + row] = 0.f;
    // per-column unscale 2^-s_r (exact), s_r from the column's max |W| (reading Q27);
    // computed once into shared memory (after the row accumulators)
    float* vscale = reinterpret_cast<float*>(smem + kRvSmem - kRvBars + 512);  // [RC] (bars use < 512 B)
    if (ew == 0 && lane < RC)
      vscale[lane] = lane < args.r_valid ? ldexpf(1.f, -rv_wcol_exp(args.wcol[args.r_off + lane])) : 0.f;
    named_bar_sync(3, 32 * kRvEpiWarps);
    int blk_next = 0;   // next V block this warp folds
    int blk_total = 0;  // V blocks issued so far (all segments before the current one)
    // fold V block `k` (lane quarter g's rows, this warp's kNC columns): wait, read, release, add
    // into the compensated FP32 accumulator (Kahan: |error| ~ 2 eps |sum|, the FP64 sum's accuracy
    // at FMA-pipe cost; FP64 converts would queue on the exponential's pipe).  The power-of-two
    // unscale is applied once, at the segment end.  V block layout: per 16 weight columns, 16
    // columns V_hh + V_lh then 16 columns V_hl.
    const uint32_t va0 = tbase + lane_off + kRvColV + (uint32_t)(32 * (rlo >> 4) + (rlo & 15));
    auto fold = [&](int k) {
      RV_WAIT(&vfull[k & 1], (uint32_t)((k >> 1) & 1), "vfull", k);
      tc_fence_after();
      const uint32_t va = va0 + (uint32_t)((k & 1) * 2 * RC);
      uint32_t vh[kNC], vl[kNC];
      float sm[kNC], cm[kNC];
      tmem_ldn<kNC>(va, vh);
      tmem_ldn<kNC>(va + 16, vl);
#pragma unroll
      for (int u = 0; u < kNC; ++u) {  // accumulator loads overlap the TMEM loads
        sm[u] = vacc[(rlo + u) * 128 + row];
        cm[u] = vcmp[(rlo + u) * 128 + row];
      }
      tmem_wait_ld();
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(&vempty[k & 1]);
#pragma unroll
      for (int u = 0; u < kNC; ++u) {
        const float x = __fadd_rn(__uint_as_float(vh[u]), __uint_as_float(vl[u]));
        const float y = __fsub_rn(x, cm[u]);
        const float t = __fadd_rn(sm[u], y);
        cm[u] = __fsub_rn(__fsub_rn(t, sm[u]), y);
        sm[u] = t;
      }
#pragma unroll
      for (int u = 0; u < kNC; ++u) {
        vacc[(rlo + u) * 128 + row] = sm[u];
        vcmp[(rlo + u) * 128 + row] = cm[u];
      }
    };
    auto vfinal = [&](int r) { return __fsub_rn(vacc[r * 128 + row], vcmp[r * 128 + row]) * vscale[r]; };
    int bq = 0, u3 = 0;
    int q = 0;
    for (int q0 = 0; q0 < count;) {
      int64_t tt;
      int st0, len;
      sc.segment(q0, tt, st0, len);
      const int seg_blocks = (len + kRvBlock - 1) / kRvBlock;
      for (int j = 0; j < len; ++j, ++q) {
        if ((q & 3) == gr) {
          RV_WAIT(&sfull[bq], (uint32_t)(u3 & 1), "sfull", q);
          if (lane == 0 && ew == 4 * gr) RV_TRACE(q, 1);
          tc_fence_after();
          // all 96 columns of the unit for this lane quarter: 6 K steps of 16 sources in three
          // 32-column batches, the next batch's load in flight while one is computed
          const uint32_t ta = tbase + lane_off + (uint32_t)(bq * kRvTS);
          uint32_t sa[32], sb[32];
          if (!(KS_DEBUG && (args.dbg & 4))) {
          tmem_ld32(ta, sa);
          tmem_wait_ld();
          tmem_ld32(ta + 32, sb);
          rv_batch<NPOLY, 32>(sa);
          if (!(KS_DEBUG && (args.dbg & 8))) tmem_st32(ta, sa);
          tmem_wait_ld();
          tmem_wait_st();  // sa is reloaded next
          tmem_ld32(ta + 64, sa);
          rv_batch<NPOLY, 32>(sb);
          if (!(KS_DEBUG && (args.dbg & 8))) tmem_st32(ta + 32, sb);
          tmem_wait_ld();
          rv_batch<NPOLY, 32>(sa);
          if (!(KS_DEBUG && (args.dbg & (8 | 32)))) tmem_st32(ta + 64, sa);  // 32: a third of P never stored
          if (!(KS_DEBUG && (args.dbg & 16))) tmem_wait_st();
          }
          tc_fence_before();
          __syncwarp();
          if (lane == 0) mbar_arrive(&pready[bq]);
          if (lane == 0 && ew == 4 * gr) RV_TRACE(q, 2);
          // fold the completed V blocks of this tile (the V issuer reuses a block's columns two
          // blocks later); one not yet complete is tried again after the next unit rather than
          // stalling the P pipeline
          {
            while (blk_next < blk_total + seg_blocks) {
              const int jl = (blk_next - blk_total) * kRvBlock;  // first unit of the block
              if (jl > j) break;
              if (!__all_sync(0xffffffffu, mbar_test(&vfull[blk_next & 1], (uint32_t)((blk_next >> 1) & 1)))) break;
              if (lane == 0 && ew == 4 * gr) RV_TRACE(q, 8);
              fold(blk_next++);
              if (lane == 0 && ew == 4 * gr) RV_TRACE(q, 9);
            }
          }
        }
        if (++bq == kRvSBufs) {
          bq = 0;
          ++u3;
        }
      }
      // ---- segment end (all epilogue warps): remaining folds, then V or a stream-K partial slot
      {
        while (blk_next < blk_total + seg_blocks) fold(blk_next++);
        const bool whole = (st0 == 0) && (len == n_s);
        const int64_t grow = tt * 128 + row;
        if (whole) {
          if (grow < args.N)
            for (int r = rlo; r < rhi; ++r)
              if (r < args.r_valid) args.V[grow * args.R + args.r_off + r] = vfinal(r);
        } else {
          const int64_t tr = tt - sc.rem_t0;
          const int slot = (tr == sc.v0 / n_s) ? 0 : 1;
          float* pp = args.partial + ((b * 2 + slot) * 128 + row) * RC;
          for (int r = rlo; r < rhi; ++r) pp[r] = vfinal(r);
          __threadfence();
          named_bar_sync(2, 32 * kRvEpiWarps);
          const int64_t b_first = rv_sk_owner(tr * n_s, sc.Urem, sc.Gr);
          const int64_t b_last = rv_sk_owner(tr * n_s + n_s - 1, sc.Urem, sc.Gr);
          if (row == 0 && gr == 0) {
            const int old = atomicAdd(&args.counters[tt], 1);
            const int lastc = (old == (int)(b_last - b_first));
            if (lastc) args.counters[tt] = 0;
            *flag = lastc;
          }
          named_bar_sync(2, 32 * kRvEpiWarps);
          if (*flag) {
            __threadfence();
            for (int r = rlo; r < rhi; ++r) {
              float sum = 0.f;
              for (int64_t bb = b_first; bb <= b_last; ++bb) {
                const int sl = (tr == rv_sk_start(bb, sc.Urem, sc.Gr) / n_s) ? 0 : 1;
                sum += __ldcg(args.partial + ((bb * 2 + sl) * 128 + row) * RC + r);
              }
              if (grow < args.N && r < args.r_valid) args.V[grow * args.R + args.r_off + r] = sum;
            }
          }
          named_bar_sync(2, 32 * kRvEpiWarps);  // flag reuse
        }
        for (int r = rlo; r < rhi; ++r) vacc[r * 128 + row] = vcmp[r * 128 + row] = 0.f;
      }
      blk_total += seg_blocks;
      q0 += len;
    }
  }

  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  if (warp == 2) tmem_dealloc(tbase, 512);
  if (args.cta_times != nullptr && threadIdx.x == 0) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    args.cta_times[4 * b + 2] = t;
    args.cta_times[4 * b + 3] = (unsigned long long)clock64();
  }
}

template <int NPOLY, int RC>
static cudaError_t launch_rv_t(const CUtensorMap* m, const RvArgs& a, cudaStream_t st) {
  static std::atomic<uint64_t> attr_done{0};
  cudaError_t e = smem_optin_once(attr_done, reinterpret_cast<const void*>(ks_fused_rv_kernel<NPOLY, RC>),
                                  (int)kRvSmem);
  if (e != cudaSuccess) return e;
  return launch_pdl(ks_fused_rv_kernel<NPOLY, RC>, a.sk.grid, kRvThreads, kRvSmem, st, m[0], m[1], m[2], m[3], m[4],
                    a);
}

// exponential pairs of 16 on the FMA pipe (KS_OPT_EXP_POLY; default 0: the P split adds ALU and
// issue work per pair; measured at K = 32, R = 16, 65,536^2: 0 / 2 / 4 / 6 -> 1.25 / 1.26 / 2.00 /
// 2.48 ms)
int rv_poly_for(int v) { return (v == 0 || v == 2 || v == 4 || v == 6) ? v : 0; }

cudaError_t launch_fused_rv(const CUtensorMap* maps, const RvArgs& a, cudaStream_t st) {
  const int np = rv_poly_for(opt(KS_OPT_EXP_POLY, -1));
  if (a.r_c == 32) {
    switch (np) {
      case 0: return launch_rv_t<0, 32>(maps, a, st);
      case 2: return launch_rv_t<2, 32>(maps, a, st);
      case 6: return launch_rv_t<6, 32>(maps, a, st);
      default: return launch_rv_t<4, 32>(maps, a, st);
    }
  }
  switch (np) {
    case 0: return launch_rv_t<0, 16>(maps, a, st);
    case 2: return launch_rv_t<2, 16>(maps, a, st);
    case 6: return launch_rv_t<6, 16>(maps, a, st);
    default: return launch_rv_t<4, 16>(maps, a, st);
  }
}

}  // namespace ks
