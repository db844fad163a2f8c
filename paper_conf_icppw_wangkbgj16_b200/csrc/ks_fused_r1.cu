// ks_fused_r1.cu -- the fused tensor-core kernel for one weight column (R = 1) with
// the norms folded into the contraction: the headline path (scope rows a2-a7).
//
// What it computes (PAPER.md SS III-C, Alg.2; Eq.1-3):
//   t_ji = sum_d bh_jd a_id + na_i + nb_j      (one tcgen05 accumulator, reading Q26)
//        = -log2(e) ||alpha_i - beta_j||^2 / (2h^2)  [+ log2(W_i / Wmax), log-weight mode]
//   V_j  = Wmax sum_i 2^t_ji                    (log-weight mode, every W_i >= 0)
//   V_j  = sum_i 2^min(t_ji, 0) W_i             (weight mode: any sign; d^2 >= 0 clamp)
// The operands are the split-FP16 planes of ks_prep (hi/lo of the power-of-2 scaled
// centred coordinates, plus six hi-plane columns carrying FP16 pieces of the norms,
// reading Q26 with the fold shift s of reading Q28); 3 products lo.hi + hi.lo + hi.hi per
// 16-column K step that holds coordinates, hi.hi for the step holding only norm pieces.
//
// Structure: one persistent 640-thread CTA per SM over (128-target x 128-source) units
// (waves of whole target tiles, then a stream-K remainder, as ks_fused_tc.cu):
//   warp 0    TMA producer: the target tile's planes once per target tile (two
//             buffers), each unit's source planes into a D-stage ring;
//   warps 1,3 MMA issuers (even / odd units): per unit 7 (K = 32) kind::f16 M=128 N=128
//             MMAs into TMEM buffer q % 4;
//   warp 2    TMEM allocation (4 x 128 columns); weight mode: each unit's 128 weights
//             into an 8-slot ring;
//   warps 4.. 16 epilogue warps in 4 groups; group g owns TMEM buffer g and every
//             unit q with q % 4 == g: tcgen05.ld 32 columns at a time (two batches in
//             flight), release the buffer once all 128 columns are in registers, then
//             exp2 (10 of 16 on MUFU.EX2, 6 as an FMA-pipe polynomial, reading Q25) and
//             FADD2 / FFMA2 row sums.  At the end of a target tile the four groups'
//             sums are combined in a fixed order; split tiles go through the stream-K
//             partial slots and a last-arriver fix-up (no atomics on V).
// Four accumulator buffers instead of two: the MMA warp can run up to three units
// ahead of the slowest group, and a group waits for its next unit only if the tensor
// pipe falls that far behind (SS6).
#include "ks_internal.h"
#include <cuda_fp16.h>
#include "ks_ptx.cuh"

// Measurement builds (never the shipped library): -DKS_DEBUG=1 honours args.dbg (work-dropping
// knobs, wrong results), -DKS_PROF=1 accumulates per-warp clock64 phase totals.
#ifndef KS_DEBUG
#define KS_DEBUG 0
#endif
#ifndef KS_PROF
#define KS_PROF 0
#endif
// -DKS_TRACE=1: CTA 0 records clock64 per unit (MMA warp: waits done / commits issued; the
// unit's group, lane quarter 0: S ready / S released) after the phase clocks (tools only)
#ifndef KS_TRACE
#define KS_TRACE 0
#endif
#if KS_TRACE
#define R1_TRACE(q, k)                                                                              \
  if (ct != nullptr && b == 0 && (q) < 4096)                                                         \
  ct[4 * args.sk.grid + 80 * args.sk.grid + 4 * (q) + (k)] = (unsigned long long)clock64()
#else
#define R1_TRACE(q, k) (void)0
#endif
#if KS_PROF
#define R1_PROF_BEGIN(v) const long long v = clock64()
#define R1_PROF_END(k, v) pf[k] += clock64() - v
#else
#define R1_PROF_BEGIN(v) (void)0
#define R1_PROF_END(k, v) (void)0
#endif

namespace ks {

namespace {

constexpr int kR1Groups = 4;                 // epilogue groups = TMEM S buffers
constexpr int kR1EpiWarps = 4 * kR1Groups;  // one warp per TMEM lane quarter per group
constexpr int kR1Threads = 128 + 32 * kR1EpiWarps;
constexpr int kR1TS = 128;                   // sources per unit
constexpr uint32_t kR1Plane = 128u * 64u;    // 128 rows x one 64-byte chunk (8 KB); 4 KB with 32-byte rows
constexpr int kR1WSlots = 8;                 // weight ring (weight mode)
constexpr int kR1MaxStages = 8;
constexpr uint32_t kR1Smem = 227u * 1024u;   // dynamic shared memory requested
constexpr uint32_t kR1Bars = 1024u;          // barriers + scratch flag at the top
constexpr uint32_t kR1Ring = kR1WSlots * 512u;
constexpr uint32_t kR1Region = kR1Smem - kR1Bars - kR1Ring - 8u * 1024u;  // operands (+ 8 KB FP64 scratch)

__device__ __forceinline__ int64_t r1_sk_start(int64_t b, int64_t U, int64_t G) { return (b * U) / G; }
__device__ __forceinline__ int64_t r1_sk_owner(int64_t u, int64_t U, int64_t G) { return ((u + 1) * G - 1) / U; }

// Persistent schedule (as ks_fused_tc.cu): `waves` full waves in which CTA b owns target tile
// w G + b and all CTAs sweep the source tiles in the same order (shared through L2), then a
// stream-K split of the remaining target tiles.
struct R1Sched {
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
      v0 = r1_sk_start(b, Urem, Gr);
      v1 = r1_sk_start(b + 1, Urem, Gr);
    }
    count = qw + (int)(v1 - v0);
  }
};
struct R1It {
  int q, st;
  int64_t tt;
};
__device__ __forceinline__ R1It r1_begin(const R1Sched& s) {
  R1It u;
  u.q = 0;
  if (s.qw > 0) {
    u.tt = s.b;
    u.st = 0;
  } else {
    u.tt = s.rem_t0 + s.v0 / s.n_s;
    u.st = (int)(s.v0 % s.n_s);
  }
  return u;
}
__device__ __forceinline__ void r1_next(const R1Sched& s, R1It& u) {
  ++u.q;
  if (u.q < s.qw) {
    if (++u.st == s.n_s) {
      u.st = 0;
      u.tt += s.G;
    }
  } else if (u.q == s.qw) {
    u.tt = s.rem_t0 + s.v0 / s.n_s;
    u.st = (int)(s.v0 % s.n_s);
  } else if (++u.st == s.n_s) {
    u.st = 0;
    ++u.tt;
  }
}

// One 32-column batch of a warp: 32 exponentials per lane, NPOLY of every 16 pairs on the
// FMA pipe (exp2_poly2, which needs t >= -125), the rest on MUFU.EX2.
//   WMUL = false (log-weight mode): acc += 2^t
//   WMUL = true  (weight mode):     acc += 2^min(t, 0) W_i   (CLAMP: the d^2 >= 0 clamp)
template <int NPOLY, bool WMUL, int CLAMP>
__device__ __forceinline__ void r1_batch(const uint32_t (&sv)[32], const float* __restrict__ w, f2_t (&acc)[2]) {
#pragma unroll
  for (int i = 0; i < 32; i += 4) {
    ulonglong2 w4;
    if constexpr (WMUL) w4 = lds_pairs(w + i);  // every lane reads the same 16 bytes (broadcast)
#pragma unroll
    for (int u = 0; u < 2; ++u) {
      const int k = (i >> 1) + u;  // pair index within the batch
      float t0 = __uint_as_float(sv[i + 2 * u]), t1 = __uint_as_float(sv[i + 2 * u + 1]);
      if constexpr (WMUL && CLAMP == 1) {  // d^2 >= 0: t <= 0
        t0 = fminf(t0, 0.f);
        t1 = fminf(t1, 0.f);
      } else if constexpr (WMUL && CLAMP == 2) {  // |d^2|: a free operand modifier of MUFU / FMNMX
        t0 = -fabsf(t0);
        t1 = -fabsf(t1);
      }
      f2_t pk;
      if (((k * NPOLY) & 15) < NPOLY) {
        pk = exp2_poly2(f2_pack(fmaxf(t0, -125.f), fmaxf(t1, -125.f)));
      } else {
        pk = f2_pack(ex2_approx(t0), ex2_approx(t1));
      }
      if constexpr (WMUL) {
        acc[k & 1] = ffma2f(pk, u ? w4.y : w4.x, acc[k & 1]);
      } else {
        acc[k & 1] = fadd2(acc[k & 1], pk);
      }
    }
  }
}

}  // namespace

// log-weight mode (device-side decision, no host sync): every W_i >= 0, max |W| > 0 and the
// host allows it (args.logw); the source prep made the same decision from the same flags.
__device__ __forceinline__ bool r1_logw(const R1Args& a) {
  return a.logw && a.wstat[1] == 0u && a.wstat[0] != 0u;
}

template <int NPOLY, int CLAMP>
__global__ void __launch_bounds__(kR1Threads, 1)
    ks_fused_r1_kernel(const __grid_constant__ CUtensorMap mA_hi, const __grid_constant__ CUtensorMap mA_lo,
                       const __grid_constant__ CUtensorMap mB_hi, const __grid_constant__ CUtensorMap mB_lo,
                       const __grid_constant__ CUtensorMap mA_f, const __grid_constant__ CUtensorMap mB_f,
                       const R1Args args) {
  extern __shared__ __align__(1024) uint8_t smem[];
  if ((smem_u32(smem) & 1023u) != 0u) __trap();  // SWIZZLE_64B atoms and descriptors assume 1 KB alignment
  // warp index through a shuffle: the compiler then treats the role branches as warp-uniform and
  // keeps the TMA/MMA warps' loop state and descriptors on the uniform datapath
  const int tid = threadIdx.x, warp = __shfl_sync(0xffffffffu, tid >> 5, 0), lane = tid & 31;
  const int64_t b = blockIdx.x;
  unsigned long long* ct = args.cta_times;
#if KS_DEBUG
  const bool dbg_noepi = args.dbg == 1 || args.dbg >= 3, dbg_nomma = args.dbg >= 2, dbg_noload = args.dbg == 4;
#else
  constexpr bool dbg_noepi = false, dbg_nomma = false, dbg_noload = false;
#endif
#if KS_PROF
  long long pf[4] = {0, 0, 0, 0};
  const long long pf_t0 = clock64();
#endif
  if (ct != nullptr && tid == 0) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    ct[4 * b] = t;
    ct[4 * b + 1] = (unsigned long long)clock64();
  }

  // ---- geometry: planes per tile (chunk 0: hi, lo; chunk 1: hi, + lo when it holds coordinates)
  const int n_kc = args.n_kc;  // operand chunks: 1 or 2 of 32 halves (64-byte rows), or 1 of 16 (narrow)
  const bool narrow = args.narrow != 0;  // K + 6 <= 16: 32-byte rows, SWIZZLE_32B, one K step
  const bool lo1 = n_kc == 2 && args.kdims > 32;
  const int P = 2 + (n_kc == 2 ? (lo1 ? 2 : 1) : 0);
  const uint32_t plane = narrow ? kR1Plane / 2 : kR1Plane;
  // fold_narrow: the fold chunk is one 16-column plane of 32-byte rows (4 KB) after the two 8 KB
  // planes of chunk 0
  const bool fnar = args.fold_narrow != 0;
  // lo_narrow: one chunk, the lo plane as 16 columns of 32-byte rows (4 KB) after the 8 KB hi plane
  const bool lnar = args.lo_narrow != 0;
  const uint32_t tile_bytes = fnar ? 2 * plane + kR1Plane / 2 : lnar ? plane + kR1Plane / 2 : (uint32_t)P * plane;
  int D = (int)((kR1Region - 2 * tile_bytes) / tile_bytes);
  if (D > kR1MaxStages) D = kR1MaxStages;
  D &= ~1;  // even: the S-MMA warp of unit q (q & 1) also issues unit q + D, so it waits on every
            // phase of a stage's full barrier (a parity wait must never skip a phase)
  const uint32_t offA = 0, offS = 2 * tile_bytes;
  uint8_t* wring = smem + kR1Region;
  double* red = reinterpret_cast<double*>(smem + kR1Region + kR1Ring);  // [4 groups][128 rows]
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem + kR1Smem - kR1Bars);
  uint64_t* full = bars;                    // [8]
  uint64_t* empty = full + kR1MaxStages;    // [8]
  uint64_t* afull = empty + kR1MaxStages;   // [2]
  uint64_t* aempty = afull + 2;             // [2]
  uint64_t* sfull = aempty + 2;             // [4]
  uint64_t* sempty = sfull + kR1Groups;     // [4]
  uint64_t* wfull = sempty + kR1Groups;     // [8]
  uint64_t* wempty = wfull + kR1WSlots;     // [8]
  uint32_t* tmem_base_smem = reinterpret_cast<uint32_t*>(wempty + kR1WSlots);
  int* flag = reinterpret_cast<int*>(tmem_base_smem + 1);

  R1Sched sc;
  sc.init(args.sk.n_t, args.sk.n_s, args.sk.grid, b);
  const int count = sc.count;
  const int n_s = sc.n_s;

  if (tid == 0) {
    for (int i = 0; i < kR1MaxStages; ++i) {
      mbar_init(&full[i], 1);
      mbar_init(&empty[i], 1);
    }
    for (int i = 0; i < 2; ++i) {
      mbar_init(&afull[i], 1);
      mbar_init(&aempty[i], 2);  // both MMA warps
    }
    for (int i = 0; i < kR1Groups; ++i) {
      mbar_init(&sfull[i], 1);
      mbar_init(&sempty[i], 4);  // the group's four warps
    }
    for (int i = 0; i < kR1WSlots; ++i) {
      mbar_init(&wfull[i], 1);
      mbar_init(&wempty[i], 4);
    }
    fence_mbar_init();
  }
  if (warp == 2) tmem_alloc(tmem_base_smem, 512);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tbase = __shfl_sync(0xffffffffu, *tmem_base_smem, 0);
  // programmatic dependent launch: the prologue above overlaps the target prep; nothing the
  // preceding kernels wrote is read before this point
  pdl_wait();
  const bool logw = r1_logw(args);

  if (warp == 0) {
    // ================= TMA producer (converged warp, one elected lane issues)
    const bool leader = elect_one();
    if (leader) {
      tma_prefetch_desc(&mA_hi);
      tma_prefetch_desc(&mB_hi);
    }
    int s = 0;
    uint32_t ph = 0;
    int seg = -1;
    int64_t cur_tt = -1;
    R1It cu = r1_begin(sc);
    for (int q = 0; q < count; ++q, r1_next(sc, cu)) {
      if (cu.tt != cur_tt) {  // new target tile: its planes into buffer seg & 1
        ++seg;
        cur_tt = cu.tt;
        const int ab = seg & 1;
        mbar_wait_uniform(&aempty[ab], (uint32_t)(((seg >> 1) & 1) ^ 1));
        if (leader) {
          uint8_t* ap = smem + offA + ab * tile_bytes;
          const int y = (int)(cu.tt * 128);
          mbar_arrive_expect_tx(&afull[ab], tile_bytes);
          tma_load_2d(ap, &mA_hi, 0, y, &afull[ab]);
          tma_load_2d(ap + plane, lnar ? &mA_f : &mA_lo, 0, y, &afull[ab]);
          if (fnar) {
            tma_load_2d(ap + 2 * plane, &mA_f, 32, y, &afull[ab]);
          } else if (n_kc == 2) {
            tma_load_2d(ap + 2 * plane, &mA_hi, 32, y, &afull[ab]);
            if (lo1) tma_load_2d(ap + 3 * plane, &mA_lo, 32, y, &afull[ab]);
          }
        }
        __syncwarp();
      }
      mbar_wait_uniform(&empty[s], ph ^ 1u);
      if (leader && dbg_noload) {
        mbar_arrive(&full[s]);
      } else if (leader) {
        uint8_t* sp = smem + offS + s * tile_bytes;
        const int y = cu.st * kR1TS;
        mbar_arrive_expect_tx(&full[s], tile_bytes);
        tma_load_2d(sp, &mB_hi, 0, y, &full[s]);
        tma_load_2d(sp + plane, lnar ? &mB_f : &mB_lo, 0, y, &full[s]);
        if (fnar) {
          tma_load_2d(sp + 2 * plane, &mB_f, 32, y, &full[s]);
        } else if (n_kc == 2) {
          tma_load_2d(sp + 2 * plane, &mB_hi, 32, y, &full[s]);
          if (lo1) tma_load_2d(sp + 3 * plane, &mB_lo, 32, y, &full[s]);
        }
      }
      __syncwarp();
      if (++s == D) {
        s = 0;
        ph ^= 1u;
      }
    }
  } else if (warp == 1 || warp == 3) {
    // ================= MMA issuers: warp 1 the even units, warp 3 the odd ones (converged warps;
    // the elected lane predicates the tcgen05 ops).  A tcgen05.mma issue blocks while the
    // tensor pipe is busy, so one warp's barrier waits for unit q + 1 overlap the other's
    // issue of unit q and the pipe sees an unbroken stream (measured: one issuing warp left
    // the pipe idle ~360 cycles per unit in its waits, SS6).
    const int mine = warp == 1 ? 0 : 1;
    const uint32_t lead = elect_one() ? 1u : 0u;
    const uint32_t idS = idesc_f16(128, kR1TS);
    // products per 16-column K step: 3 (coordinates: lo.hi, hi.lo, hi.hi), 1 (norm pieces only), 0
    uint32_t plan = 0;
    for (int st4 = 0; st4 < (narrow ? 1 : 2 * n_kc); ++st4) {
      const int col0 = st4 * 16;
      const uint32_t np = col0 >= args.kcols ? 0u : (col0 >= args.kdims ? 1u : 3u);
      plan |= np << (2 * st4);
    }
    // descriptors: low words (start address >> 4) advance within the same high word
    const uint32_t dhi = (uint32_t)((narrow ? sdesc_k_sw32(smem) : sdesc_k_sw64(smem)) >> 32);
    const uint32_t dhi1 = fnar ? (uint32_t)(sdesc_k_sw32(smem) >> 32) : dhi;  // chunk 1's layout
    const uint32_t dhiL = lnar ? (uint32_t)(sdesc_k_sw32(smem) >> 32) : dhi;  // the lo plane's layout
    const uint32_t dA0 = (uint32_t)sdesc_k_sw64(smem + offA), dS0 = (uint32_t)sdesc_k_sw64(smem + offS);
    const uint32_t kP16 = plane >> 4;
    const uint32_t tile16 = tile_bytes >> 4;
    int s = 0;
    uint32_t ph = 0;
    int seg = -1;
    int64_t cur_tt = -1;
    R1It cu = r1_begin(sc);
    for (int q = 0; q < count; ++q, r1_next(sc, cu)) {
      const int bq = q & (kR1Groups - 1);
      if (cu.tt != cur_tt) {  // new target tile: release the previous buffer, wait for this one
        if (seg >= 0) tc_commit_if(&aempty[seg & 1], lead);
        ++seg;
        cur_tt = cu.tt;
        mbar_wait_uniform(&afull[seg & 1], (uint32_t)((seg >> 1) & 1));
      }
      if ((q & 1) != mine) {  // the other warp's unit: only the stage counter advances
        if (++s == D) {
          s = 0;
          ph ^= 1u;
        }
        continue;
      }
      R1_PROF_BEGIN(w0);
      if (q >= kR1Groups) mbar_wait_uniform(&sempty[bq], (uint32_t)(((q >> 2) - 1) & 1));  // group bq read unit q - 4
      R1_PROF_END(0, w0);
      R1_PROF_BEGIN(w1);
      mbar_wait_uniform(&full[s], ph);
      R1_PROF_END(1, w1);
      if (lane == 0) R1_TRACE(q, 0);
      R1_PROF_BEGIN(w2);
      tc_fence_after();
      const uint32_t dS = tbase + (uint32_t)(bq * kR1TS);
      const uint32_t aT = dA0 + (uint32_t)(seg & 1) * tile16, bT = dS0 + (uint32_t)s * tile16;
#pragma unroll
      for (int kc = 0; kc < 2; ++kc) {
        if (kc >= n_kc) break;
        const uint32_t pl = kc == 0 ? 0u : 2u;  // first plane of chunk kc
        const uint32_t aH = aT + pl * kP16, aL = aH + kP16, bH = bT + pl * kP16, bL = bH + kP16;
#pragma unroll
        for (int ks = 0; ks < 2; ++ks) {
          const uint32_t np = (plan >> (2 * (2 * kc + ks))) & 3u;
          const uint32_t o = (uint32_t)(ks * 2);  // 32 bytes along K
          const uint32_t acc0 = (kc > 0 || ks > 0) ? 1u : 0u;
          if (dbg_nomma) {
          } else if (np == 3u) {  // small terms first
            if (lnar) {  // lo planes in the 32-byte-row layout (ks = 0 only: columns 0..15)
              mma_f16_lo2(dS, aL, dhiL, bH, dhi, idS, acc0, lead);
              mma_f16_lo2(dS, aH, dhi, bL, dhiL, idS, 1u, lead);
            } else {
              mma_f16_lo(dS, aL + o, bH + o, dhi, idS, acc0, lead);
              mma_f16_lo(dS, aH + o, bL + o, dhi, idS, 1u, lead);
            }
            mma_f16_lo(dS, aH + o, bH + o, dhi, idS, 1u, lead);
          } else if (np == 1u) {
            mma_f16_lo(dS, aH + o, bH + o, kc == 0 ? dhi : dhi1, idS, acc0, lead);
          }
        }
      }
      tc_commit_if(&empty[s], lead);
      tc_commit_if(&sfull[bq], lead);
      R1_PROF_END(2, w2);
      if (lane == 0) R1_TRACE(q, 1);
      if (++s == D) {
        s = 0;
        ph ^= 1u;
      }
    }
  } else if (warp == 2) {
    // ================= weight-mode producer: the unit's 128 weights (512 B) into the ring
    if (!logw) {
      const bool leader = elect_one();
      R1It cu = r1_begin(sc);
      for (int q = 0; q < count; ++q, r1_next(sc, cu)) {
        const int slot = q % kR1WSlots;
        mbar_wait(&wempty[slot], (uint32_t)(((q / kR1WSlots) & 1) ^ 1));
        if (leader) {
          mbar_arrive_expect_tx(&wfull[slot], 512u);
          bulk_load(wring + slot * 512, args.wv + (int64_t)cu.st * kR1TS, 512u, &wfull[slot]);
        }
        __syncwarp();
      }
    }
  } else if (warp >= 4) {
    // ================= epilogue: group gr (TMEM buffer gr), lane quarter g
    const int ew = warp - 4;
    const int g = ew & 3, gr = ew >> 2;
    const int row = 32 * g + lane;
    const uint32_t ta = tbase + ((uint32_t)(32 * g) << 16) + (uint32_t)(gr * kR1TS);
    f2_t acc[2] = {0ull, 0ull};
    float vhi = 0.f, vlo = 0.f;  // unevaluated FP32 pair (TwoSum folds, exact)
    int nblk = 0;
    auto fold = [&]() {
      float a0, a1, a2, a3;
      f2_unpack(acc[0], a0, a1);
      f2_unpack(acc[1], a2, a3);
      const float blk = (a0 + a1) + (a2 + a3);
      acc[0] = acc[1] = 0ull;
      const float sum = vhi + blk;
      const float bb = sum - vhi;
      vlo += (vhi - (sum - bb)) + (blk - bb);
      vhi = sum;
    };
    // segments (runs of units of one target tile) computed once each, so the unit loop keeps
    // only q and the segment end live
    for (int q = 0; q < count;) {
      int64_t tt;
      int st0, len;
      if (q < sc.qw) {
        tt = b + (int64_t)(q / n_s) * sc.G;
        st0 = 0;
        len = n_s;
      } else {
        const int64_t v = sc.v0 + (q - sc.qw);
        tt = sc.rem_t0 + v / n_s;
        st0 = (int)(v % n_s);
        len = n_s - st0 < count - q ? n_s - st0 : count - q;
      }
      const int q_end = q + len;
      for (int qq = q + ((gr - q) & (kR1Groups - 1)); qq < q_end; qq += kR1Groups) {
        R1_PROF_BEGIN(e0);
        mbar_wait(&sfull[gr], (uint32_t)((qq >> 2) & 1));
        R1_PROF_END(0, e0);
        if (lane == 0 && g == 0) R1_TRACE(qq, 2);
        R1_PROF_BEGIN(e1);
        tc_fence_after();
        const int slot = qq % kR1WSlots;
        if (!logw) mbar_wait(&wfull[slot], (uint32_t)((qq / kR1WSlots) & 1));
        const float* w = reinterpret_cast<const float*>(wring + slot * 512);
        uint32_t sa[32], sb[32];
        tmem_ld32(ta, sa);
        tmem_wait_ld();
        tmem_ld32(ta + 32, sb);
        if (dbg_noepi) acc[0] ^= sa[0] ^ sa[31];
        else if (logw) r1_batch<NPOLY, false, false>(sa, w, acc);
        else r1_batch<NPOLY, true, CLAMP>(sa, w, acc);
        tmem_wait_ld();
        tmem_ld32(ta + 64, sa);
        if (dbg_noepi) acc[0] ^= sb[0] ^ sb[31];
        else if (logw) r1_batch<NPOLY, false, false>(sb, w + 32, acc);
        else r1_batch<NPOLY, true, CLAMP>(sb, w + 32, acc);
        tmem_wait_ld();
        tmem_ld32(ta + 96, sb);
        tmem_wait_ld();
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(&sempty[gr]);  // the MMA warp may overwrite the buffer
        if (lane == 0 && g == 0) R1_TRACE(qq, 3);
        if (dbg_noepi) {
          acc[1] ^= sa[0] ^ sb[31];
          if (!logw) {
            __syncwarp();
            if (lane == 0) mbar_arrive(&wempty[slot]);
          }
        } else if (logw) {
          r1_batch<NPOLY, false, false>(sa, w + 64, acc);
          r1_batch<NPOLY, false, false>(sb, w + 96, acc);
        } else {
          r1_batch<NPOLY, true, CLAMP>(sa, w + 64, acc);
          r1_batch<NPOLY, true, CLAMP>(sb, w + 96, acc);
          __syncwarp();
          if (lane == 0) mbar_arrive(&wempty[slot]);
        }
        if (++nblk == 4) {  // FP32 over <= 4 of this group's units (512 terms in 4 lanes), then TwoSum
          fold();
          nblk = 0;
        }
        R1_PROF_END(1, e1);
      }
      R1_PROF_BEGIN(e2);
      // ---- segment end: the four groups' row sums in a fixed order, then V or a partial slot
      fold();
      nblk = 0;
      const bool whole = (st0 == 0) && (len == n_s);
      const int64_t grow = tt * 128 + row;
      const double wsc = logw ? (double)__uint_as_float(args.wstat[0]) : 1.0;
      red[gr * 128 + row] = ((double)vhi + (double)vlo) * wsc;
      vhi = vlo = 0.f;
      named_bar_sync(1, 32 * kR1EpiWarps);
      if (gr == 0) {
        const double v = ((red[row] + red[128 + row]) + red[256 + row]) + red[384 + row];
        if (whole) {
          if (grow < args.N) args.V[grow] = (float)v;
        } else {
          const int64_t tr = tt - sc.rem_t0;
          const int slot = (tr == sc.v0 / n_s) ? 0 : 1;
          args.partial[(b * 2 + slot) * 128 + row] = (float)v;
          __threadfence();
          named_bar_sync(2, 128);
          const int64_t b_first = r1_sk_owner(tr * n_s, sc.Urem, sc.Gr);
          const int64_t b_last = r1_sk_owner(tr * n_s + n_s - 1, sc.Urem, sc.Gr);
          if (row == 0) {
            const int old = atomicAdd(&args.counters[tt], 1);
            const int last = (old == (int)(b_last - b_first));
            if (last) args.counters[tt] = 0;
            *flag = last;
          }
          named_bar_sync(2, 128);
          if (*flag) {
            __threadfence();
            float sum = 0.f;
            for (int64_t bb = b_first; bb <= b_last; ++bb) {
              const int sl = (tr == r1_sk_start(bb, sc.Urem, sc.Gr) / n_s) ? 0 : 1;
              sum += __ldcg(args.partial + (bb * 2 + sl) * 128 + row);
            }
            if (grow < args.N) args.V[grow] = sum;
          }
          named_bar_sync(2, 128);  // flag reuse
        }
      }
      named_bar_sync(1, 32 * kR1EpiWarps);  // red reuse
      R1_PROF_END(2, e2);
      q = q_end;
    }
  }

#if KS_PROF
  pf[3] = clock64() - pf_t0;  // this warp's run (before the final barrier)
  if (ct != nullptr && lane == 0)
    for (int k = 0; k < 4; ++k) ct[4 * args.sk.grid + (b * 20 + warp) * 4 + k] = (unsigned long long)pf[k];
#endif
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  if (warp == 2) tmem_dealloc(tbase, 512);
  if (ct != nullptr && tid == 0) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    ct[4 * b + 2] = t;
    ct[4 * b + 3] = (unsigned long long)clock64();
  }
}

// exponential pairs of 16 on the FMA pipe (KS_OPT_EXP_POLY tuning option; default measured)
int r1_poly_for(int v) { return (v == 0 || v == 4 || v == 5 || v == 6 || v == 7 || v == 8) ? v : 6; }
int r1_poly() { return r1_poly_for(opt(KS_OPT_EXP_POLY, -1)); }

template <int NPOLY, int CLAMP>
static cudaError_t launch_r1_t(const CUtensorMap* m, const R1Args& a, cudaStream_t st) {
  static std::atomic<uint64_t> attr_done{0};
  cudaError_t e = smem_optin_once(attr_done, reinterpret_cast<const void*>(ks_fused_r1_kernel<NPOLY, CLAMP>),
                                  (int)kR1Smem);
  if (e != cudaSuccess) return e;
  return launch_pdl(ks_fused_r1_kernel<NPOLY, CLAMP>, a.sk.grid, kR1Threads, kR1Smem, st, m[0], m[1], m[2], m[3], m[4],
                    m[5], a);
}

cudaError_t launch_fused_r1(const CUtensorMap* maps, const R1Args& a, int npoly, cudaStream_t st) {
  if (a.clamp == 2) return npoly == 4 ? launch_r1_t<4, 2>(maps, a, st) : launch_r1_t<6, 2>(maps, a, st);
  if (a.clamp == 1) {
    switch (npoly) {
      case 0: return launch_r1_t<0, 1>(maps, a, st);
      case 4: return launch_r1_t<4, 1>(maps, a, st);
      case 5: return launch_r1_t<5, 1>(maps, a, st);
      default: return launch_r1_t<6, 1>(maps, a, st);
    }
  }
  switch (npoly) {
    case 0: return launch_r1_t<0, 0>(maps, a, st);
    case 4: return launch_r1_t<4, 0>(maps, a, st);
    case 5: return launch_r1_t<5, 0>(maps, a, st);
    case 7: return launch_r1_t<7, 0>(maps, a, st);
    case 8: return launch_r1_t<8, 0>(maps, a, st);
    default: return launch_r1_t<6, 0>(maps, a, st);
  }
}

int fused_r1_stages(int K, bool narrow_planes) {
  const int n_kc = K + 6 <= 32 ? 1 : 2;
  const int P = 2 + (n_kc == 2 ? (K > 32 ? 2 : 1) : 0);
  const bool fnar = narrow_planes && K + 6 > 32 && K <= 32, lnar = narrow_planes && K + 6 > 16 && K <= 16;
  const uint32_t tb = fnar ? 2 * kR1Plane + kR1Plane / 2
                      : lnar ? kR1Plane + kR1Plane / 2
                             : (uint32_t)P * (K + 6 <= 16 ? kR1Plane / 2 : kR1Plane);
  int d = (int)((kR1Region - 2 * tb) / tb);
  return d > kR1MaxStages ? kR1MaxStages : d;
}

}  // namespace ks
