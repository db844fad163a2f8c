// ks_internal.h -- host-side declarations shared by the C-ABI layer and the
// kernel translation units (not part of the public ABI).
#pragma once

#include <cuda.h>
#include <cuda_runtime.h>
#include <atomic>
#include <cstdint>

#include "ks.h"

namespace ks {

// Programmatic dependent launch (PDL): kernels of the TC path after the source statistics are
// launched with programmatic stream serialization, start their CTAs while the preceding
// kernel finishes (it calls pdl_trigger early) and block in pdl_wait until it has completed
// and its writes are visible; every such kernel calls pdl_wait before touching memory the
// preceding kernels write or read.  KS_PDL=0 launches them plainly (measurement knob).
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }
bool pdl_enabled();
template <typename... KArgs, typename... Args>
cudaError_t launch_pdl(void (*kernel)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t st,
                       Args&&... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = pdl_enabled() ? 1 : 0;
  return cudaLaunchKernelEx(&cfg, kernel, static_cast<KArgs>(args)...);
}

// The dynamic shared-memory opt-in (cudaFuncAttributeMaxDynamicSharedMemorySize) is per device:
// set it once per (kernel instantiation, device).  `done` is a per-instantiation bitmask of
// device ordinals (devices >= 64 set it on every launch).
inline cudaError_t smem_optin_once(std::atomic<uint64_t>& done, const void* fn, int bytes) {
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  const uint64_t bit = dev < 64 ? (1ull << dev) : 0ull;
  if (bit && (done.load(std::memory_order_acquire) & bit)) return cudaSuccess;
  e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
  if (e == cudaSuccess && bit) done.fetch_or(bit, std::memory_order_acq_rel);
  return e;
}

// Tuning options of the context making the current API call (ks_set_option, include/ks.h),
// visible to the kernel launchers for the duration of that call.
struct Opts {
  int v[KS_OPT_COUNT_];
};
extern thread_local const Opts* tl_opts;
inline int opt(int id, int dflt) { return tl_opts ? tl_opts->v[id] : dflt; }

constexpr int kTileT = 256;   // targets per CTA tile (FP32 path)
constexpr int kTileS = 128;   // sources per pipeline stage (FP32 path)
constexpr int kFp32Threads = 512;  // 16 warps, one CTA per SM

// Stream-K partition of the (target tile x source tile) unit space over G
// persistent CTAs: CTA b owns units [b*U/G, (b+1)*U/G).
struct StreamK {
  int64_t units;       // U = n_t * n_s
  int64_t n_t;         // target tiles
  int32_t n_s;         // source tiles
  int32_t grid;        // G
};

// ---------------------------------------------------------------- prep (a1)
// mu[d] (FP32, d < k_pad; zero for d >= K) = mean_i alpha[i][d], FP64 accumulation, fixed order.
// Source statistics, one launch (ks_prep.cu): mu [k_pad] (FP32 mean, 0 for
// padding dims); if amax != nullptr its FP32 bits of max |alpha - mu|; if W !=
// nullptr (R = 1) wstat = {bits of max |W_i|, any W_i < 0 or NaN}.  Scratch:
// part [nparts][K] doubles, pmm [nparts][K][2] floats, pw [nparts][2]; counter
// must be zero before the first call and is left zero.
cudaError_t launch_source_stats(const float* alpha, const float* W, int64_t M, int K, int k_pad, int nparts,
                                double* part, float* pmm, unsigned* pw, unsigned* counter, float* mu,
                                unsigned* amax, unsigned* wstat, cudaStream_t st);

// FP32 path source layout, dimension-major [k_pad + 2][m_pad]:
//   rows d < k_pad : a[d][i]  = RN(2c * (alpha[i][d] - mu[d]))
//   row k_pad      : na[i]    = RN(-c * ||alpha_i - mu||^2)   (FP64 accumulation)
//   row k_pad + 1  : W[i]     (0 for padding)
cudaError_t launch_prep_fp32(const float* alpha, const float* W, int64_t M, int64_t m_pad, int K, int k_pad,
                             const float* mu, double c, float* src, cudaStream_t st);

// ---------------------------------------------------------------- FP32 fused kernel (a2-a7)
struct Fp32Args {
  const float* beta;   // [N][K] raw targets
  int64_t N;
  int K;
  const float* mu;     // [k_pad]
  double c;            // log2(e) / (2 h^2)
  float* V;            // [N]
  float* partial;      // [grid][2][kTileT]
  int* counters;       // [n_t], zero on entry, left zero on exit
  StreamK sk;
  unsigned long long* cta_times;  // debug: [grid][2] globaltimer at CTA start / end, or nullptr
};

// Returns the number of stages used; launches one kernel.
cudaError_t launch_fused_fp32(const CUtensorMap* tmap_src, int k_pad, const Fp32Args& a, cudaStream_t st);
int fused_fp32_ctas_per_sm(int k_pad);
int fused_fp32_stages(int k_pad);

}  // namespace ks

namespace ks {

// ---------------------------------------------------------------- tensor-core (tcgen05) path
constexpr int kTcTileT = 128;  // targets per tile = MMA M = TMEM lanes
constexpr int kTcTileS = 128;  // sources per tile = N of the S MMA = K of the V MMA
constexpr int kRvTileS = 96;   // sources per unit of the R > 1 kernel (ks_fused_rv.cu)
constexpr int kTcKC = 16;      // K floats per pipeline stage (64-byte rows, SWIZZLE_64B)
constexpr int kTcEpiWarps = 16;  // epilogue warps (4 per TMEM lane group)
constexpr int kTcThreads = 128 + 32 * kTcEpiWarps;  // warp 0 operand TMA, 1 MMA, 2 TMEM alloc, 3 norms/weights loads, 4.. epilogue

struct TcArgs {
  int64_t N;            // targets
  int k_pad;            // multiple of kTcKC
  int r_c;              // weight columns handled by this launch (16 or 32)
  int r_valid;          // valid columns among them
  int r_off;            // first weight column of this launch
  int R;                // row stride of V
  int three;            // 1: three split products (hi.hi + hi.lo + lo.hi), 0: plain TF32 (hi.hi)
  int f16;              // 1: operands are the FP16 split of power-of-2 scaled values (kind::f16 MMA)
  const float* tsc;     // [n_pad] per-target factor on S: 1 (TF32 modes) or 2^-(eA+eB_j) (FP16 mode)
  const unsigned* wstat;  // R = 1: {bits of max |W|, any W < 0}; na holds log-weights when W >= 0; else nullptr
  int aug;              // 1: norms folded into the contraction (2 extra K columns), epilogue adds nothing
  int kcols;            // operand columns (elements) that can be nonzero: MMA K steps at or past it are skipped
  int kdims;            // columns that need every split product; steps holding only [kdims, kcols) run hi.hi
  int fold;             // FP16, R = 1: folded layout (norms + log-weight in 6 hi-plane columns); active on the
                        // device iff f16_fold_ok(amax, c, K) (prep and kernel evaluate the same test)
  const unsigned* amax; // FP16: bits of max |alpha - mu|
  double c;             // log2(e) / (2 h^2)
  int K;
  int vcc;              // RV > 0: weighted sum on CUDA cores over RV padded columns (no W^T tiles, no V MMA)
  const float* wv;      // [m_pad][RV] weights, zero padded (vcc)
  const unsigned* wcol; // FP16 V-MMA (f16, !vcc): [r_pad] FP32 bits of max_i |W_ir| (column scale exponents)
  int wslots;           // VCC W/na ring depth (2..4; 0 = default)
  int ares;             // R = 1, <= 2 operand chunks: target operand resident per target tile (no reload per unit)
  int ar_stages;        // FP16 V-MMA, resident target operand: source stages (4; 5 measurement knob)
  int dbg_skip_v;       // measurement only (KS_TC_DEBUG_SKIP_V=1): do not issue the V MMAs (wrong results)
  const float* na;      // [m_pad]  -c ||alpha_hat||^2
  const float* nb;      // [n_pad]  -c ||beta_hat||^2
  float* V;             // [N][R]
  float* partial;       // [grid][2][kTcTileT][r_c]
  int* counters;        // [n_t]
  StreamK sk;
  unsigned long long* cta_times;
};

// ---------------------------------------------------------------- R = 1 folded kernel (ks_fused_r1.cu)
// Split-FP16 operands with the norms folded into the contraction (K + 6 <= 64), one weight
// column.  Sources in 128-row tiles (box rows 128 for both operand maps).
struct R1Args {
  int64_t N;              // targets
  int n_kc;               // 64-byte operand chunks (32 halves each): 1 or 2
  int narrow;             // K + 6 <= 16: one chunk of 16 halves (32-byte rows, SWIZZLE_32B maps)
  int kdims;              // coordinate columns (= K): K steps below need all three split products
  int kcols;              // K + 6: steps at or past it are zero padding
  int logw;               // host allows the log-weight mode (decided on the device from wstat)
  int clamp;              // weight mode: 1 clamp t <= 0 (d^2 >= 0) before the exponential, 2 t -> -|t|
  const unsigned* wstat;  // {bits of max |W|, any W < 0 or NaN}
  const float* wv;        // [m_pad] raw weights, zero padded (weight mode)
  float* V;               // [N]
  float* partial;         // [grid][2][128]
  int* counters;          // [n_t], zero on entry, left zero
  StreamK sk;             // n_s = m_pad / 128
  unsigned long long* cta_times;  // debug: [grid][4] globaltimer, clock64 at CTA start; the same at the end
                                  // (KS_PROF builds: then [grid][20 warps][4] per-warp phase clocks)
  int dbg;                // KS_DEBUG builds only (KS_R1_DEBUG): 1 no epilogue math, 2 no MMAs, 3 neither, 4 + no source loads
  int fold_narrow;        // the second chunk holds only the folded norm pieces (K <= 32, K + 6 <= 48):
                          // it is loaded as ONE 16-column plane with 32-byte rows (maps 4, 5,
                          // SWIZZLE_32B) instead of a 64-byte chunk -- a sixth fewer operand bytes
  int lo_narrow;          // one chunk, K <= 16 < K + 6: the lo plane's columns 16..31 are never
                          // multiplied -- it loads as a 16-column plane of 32-byte rows (maps 4, 5
                          // over the lo arrays), a quarter fewer operand bytes
};
// maps: A_hi, A_lo (targets), B_hi, B_lo (sources), then 32-byte-row boxes read only with
// fold_narrow (the hi planes' columns 32..47) or lo_narrow (the lo planes' columns 0..15)
cudaError_t launch_fused_r1(const CUtensorMap* maps, const R1Args& a, int npoly, cudaStream_t st);

// ---------------------------------------------------------------- R > 1 folded kernel (ks_fused_rv.cu)
// Split-FP16, K + 6 <= 64, weights as the FP16 V-MMA's wcat (launch_prep_wcat); r_c = 16 or 32
// weight columns per launch.  maps: A_hi, A_lo, B_hi, B_lo (128-row boxes), wcat (encode_wcat).
struct RvArgs {
  int64_t N;
  int n_kc, narrow, kdims, kcols;
  int r_c, r_off, r_valid, R;  // columns of this launch, first column, valid ones, V row stride
  const unsigned* wcol;        // [r_pad] FP32 bits of max_i |W_ir| (column scale exponents)
  float* V;                    // [N][R]
  float* partial;              // [grid][2][128][r_c]
  int* counters;               // [n_t]
  StreamK sk;
  unsigned long long* trace;   // KS_TRACE builds: [4096][12] unit clocks of CTA 0, or nullptr
  int dbg;                     // KS_DEBUG builds: work-dropping bits (ks_fused_rv.cu), else 0
  unsigned long long* cta_times;  // KS_OPT_MEASURE_CLOCK: [grid][4] globaltimer / clock64 at start, end
};
cudaError_t launch_fused_rv(const CUtensorMap* maps, const RvArgs& a, cudaStream_t st);
int rv_poly_for(int opt_value);
int fused_r1_stages(int K, bool narrow_planes);
int r1_poly();
int r1_poly_for(int opt_value);  // the NPOLY the R = 1 kernel runs for a KS_OPT_EXP_POLY value

// sources: src_hi/lo [m_pad][k_pad] = TF32 split of RN(2c (alpha - mu)),
// na [m_pad], W^T split wt_hi/lo [r_pad][m_pad] (zero padded)
// aug: columns K, K+1 hold (1, na_i) so that S already contains the norms
cudaError_t launch_prep_tc_sources(const float* alpha, const float* W, int64_t M, int64_t m_pad, int K, int k_pad,
                                   int R, int r_pad, const float* mu, double c, int aug, float* src_hi,
                                   float* src_lo, float* na, float* wt_hi, float* wt_lo, float* wv, int rv,
                                   const unsigned* wstat, cudaStream_t st);
// targets: tgt_hi/lo [n_pad][k_pad] = TF32 split of (beta - mu), nb [n_pad]
// aug: columns K, K+1 hold (nb_j, 1)
cudaError_t launch_prep_tc_targets(const float* beta, int64_t N, int64_t n_pad, int K, int k_pad, const float* mu,
                                   double c, int aug, float* tgt_hi, float* tgt_lo, float* nb, float* tsc,
                                   cudaStream_t st);
// FP16 mode (KS_PREC_3XF16).  k_pad is a multiple of 2*kTcKC halves (one
// 64-byte row chunk per stage, as in TF32 mode).  amax = max |alpha - mu|
// (FP32 bits, from launch_source_stats).  Sources are scaled by
// sA = 2^(13 - e), e = exponent of RN(2c * amax) (frexp convention), targets
// per row by sB_j = 2^(13 - e_j) from max_k |beta_jk - mu_k|; each scaled
// value x is split x = hi + lo, hi = RN_f16(x), lo = RN_f16(x - hi);
// tsc[j] = 2^-(log2 sA + log2 sB_j) undoes the scaling on S.
// R = 1 weight statistics (launch_source_stats): wstat[0] = FP32 bits of max |W_i|,
// wstat[1] = 1 if any W_i < 0.  With W >= 0 and max > 0 the source prep stores na_i + log2(W_i / max) in na
// (-inf for W_i = 0) and the fused kernel sums 2^t, scaling by max at the end.
// fold = 1 (R = 1): folded layout, k_pad >= K + 6 -- columns K..K+5 carry the
// norms (and log-weights) as FP16 pieces when c K amax^2 <= 2^12 (checked on
// the device); operands are then scaled by 2^eF / 2^-eF and tsc = 1, nb = na = 0.
cudaError_t launch_prep_f16_sources(const float* alpha, const float* W, int64_t M, int64_t m_pad, int K, int k_pad,
                                    int R, int r_pad, const float* mu, double c, const unsigned* amax, int fold,
                                    void* src_hi, void* src_lo, float* na, float* wt_hi, float* wt_lo, float* wv,
                                    int rv, const unsigned* wstat, cudaStream_t st);
// Folded layouts (fold 2, 3; k_pad in {16, 32, 64}, K + 6 <= k_pad): the source statistics (mu,
// amax, and wstat when non-null) and the folded source prep in one cooperative launch of `grid`
// blocks (coop_prep_grid; scratch part [grid][K], pmm [grid][K][2], pw [grid][2]; bar [2] zero
// when allocated, left zero by every launch).  Same outputs as launch_source_stats + launch_prep_f16_sources.
int coop_prep_grid(int k_pad, int64_t m_pad, int num_sms);
cudaError_t launch_prep_fold_sources_coop(const float* alpha, const float* W, int64_t M, int64_t m_pad, int K,
                                          int k_pad, int R, double c, int fold, int grid, double* part, float* pmm,
                                          unsigned* pw, unsigned* bar, float* mu, unsigned* amax, unsigned* wstat,
                                          void* src_hi, void* src_lo, float* na, float* wv, int rv, cudaStream_t st);
cudaError_t launch_prep_f16_targets(const float* beta, int64_t N, int64_t n_pad, int K, int k_pad, const float* mu,
                                    double c, const unsigned* amax, int fold, void* tgt_hi, void* tgt_lo, float* nb,
                                    float* tsc, cudaStream_t st);
// FP16 V-MMA weights (f16 mode, R > RV limit or forced): wcol [R] = bits of max_i |W_ir|
// (scratch pcol [nparts][R], counter zero before, left zero), wcat [2 r_pad][m_pad] halves
// (row 32g + u = hi of column 16g + u scaled by 2^s_r, row 32g + 16 + u = lo).
cudaError_t launch_prep_wcat(const float* W, int64_t M, int64_t m_pad, int R, int r_pad, int nparts, unsigned* pcol,
                             unsigned* counter, unsigned* wcol, void* wcat, cudaStream_t st);
// maps: A_hi, A_lo (targets), B_hi, B_lo (sources), W_hi, W_lo (weights^T)
cudaError_t launch_fused_tc(const CUtensorMap* maps, const TcArgs& a, cudaStream_t st);
int fused_tc_stages(int vcc, bool f16, int k_pad_f32, int r_c);
int fused_tc_tile_s(int rv);  // sources per tile: 256 with the CUDA-core weighted sum, 128 otherwise
int fused_tc_rv(int R);       // padded weight columns of the CUDA-core weighted sum, 0 if R > 16
size_t fused_tc_smem(int r_c);

}  // namespace ks
