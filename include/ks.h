/*
 * ks.h -- C ABI of libks.so: fused Gaussian kernel summation on NVIDIA B200
 * (sm_100a).
 *
 * The library evaluates, for sources alpha_i in R^K with weights W_i in R^R
 * and targets beta_j in R^K,
 *
 *     V[j][r] = sum_{i<M} exp( -||alpha_i - beta_j||^2 / (2 h^2) ) * W[i][r]
 *
 * i.e. Eq.1 + Eq.2 of Wang et al., "Optimizing GPGPU Kernel Summation for
 * Performance and Energy Efficiency", ICPP Workshops 2016 (PAPER.md P:L24-38,
 * SS I), with the squared distance taken through the norm identity Eq.3
 * and the -2 alpha^T beta contraction, the norm add, the exp and
 * the weighted reduction fused in one kernel so the M x N kernel matrix never
 * reaches memory (SS III-C, Alg.2).  Readings of the paper
 * (which set carries W, the 2h^2 bandwidth, M != N, R columns) are listed
 * in DESIGN.md SS3.
 *
 * Conventions (all entry points):
 *   - extern "C", no C++ exceptions cross the boundary, no torch types.
 *   - Arrays are FP32, row-major, one point's K coordinates contiguous
 *     (A row-major / B column-major in the paper's GEMM view).
 *   - Pointers taken by ks_set_sources / ks_eval are CUDA DEVICE pointers on
 *     the context's device; the *_host variants take HOST pointers.
 *   - Every call returns a ks_status.  On failure nothing is enqueued, the
 *     context is unchanged, and ks_last_error() holds a thread-local detail
 *     string.  There is no CPU fallback: without a usable sm_100 device,
 *     ks_create fails with KS_ECUDA / KS_EUNSUPPORTED.
 *   - Threading: a context is used by one host thread at a time.  Distinct
 *     contexts are independent.
 */
#ifndef KS_H_
#define KS_H_

#include <stdint.h>

#if defined(__GNUC__)
#define KS_API __attribute__((visibility("default")))
#else
#define KS_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

typedef struct ks_ctx ks_ctx;

typedef enum {
  KS_OK = 0,
  KS_EINVAL = 1,        /* bad argument (size, NULL, h, K, R)                */
  KS_ESTATE = 2,        /* ks_eval before ks_set_sources                     */
  KS_ENOMEM = 3,        /* device allocation failed                          */
  KS_ECUDA = 4,         /* CUDA runtime / launch error (see ks_last_error)   */
  KS_EUNSUPPORTED = 5   /* no kernel for this (K, R, precision) or no sm_100 */
} ks_status;

typedef enum {
  KS_PREC_AUTO = 0,     /* 3XF16 (the tcgen05 path) for every shape          */
  KS_PREC_FP32 = 1,     /* FP32 FFMA2 contraction (K <= 32, R == 1)          */
  KS_PREC_3XTF32 = 2,   /* tcgen05 tensor cores, TF32 hi/lo split, 3 products */
  KS_PREC_TF32 = 3,     /* tcgen05 tensor cores, single TF32 product         */
  KS_PREC_3XF16 = 4     /* tcgen05 tensor cores, FP16 hi/lo split of power-of-2
                           scaled operands, 3 products (same 22-bit operand
                           precision as 3XTF32 at twice the MMA rate)        */
} ks_precision;

typedef enum { KS_PATH_NONE = 0, KS_PATH_FP32 = 1, KS_PATH_TC = 2 } ks_path;

/* Launch/plan description of the last configured path (for reports). */
typedef struct {
  int path;             /* ks_path chosen for the current sources            */
  int precision;        /* effective ks_precision (never AUTO)               */
  int k_pad;            /* K padded to the kernel's dimension granularity    */
  int tile_t;           /* targets per CTA tile                              */
  int tile_s;           /* sources per pipeline stage                        */
  int num_ctas;         /* persistent CTAs of the last ks_eval launch        */
  int stages;           /* TMA pipeline depth                                */
  int num_sms;          /* SMs of the device                                 */
  int64_t m;            /* sources currently set                             */
  int64_t m_pad;        /* padded source count                               */
  int r;                /* weight columns                                    */
  int64_t launches;     /* cumulative kernels launched by this context       */
  int64_t fused_launches; /* cumulative launches of the fused kernel         */
  double c_log2;        /* c = log2(e) / (2 h^2), the ex2 prescale           */
  int kernel;           /* 0 none, 1 FP32 kernel, 2 general tcgen05 kernel,
                           3 R = 1 tcgen05 kernel (ks_fused_r1.cu),
                           4 R > 1 tcgen05 kernel (ks_fused_rv.cu)            */
  int exp_poly;         /* exponential pairs of every 16 on the FMA pipe      */
  int r1_epilogue;      /* R = 1 kernel: KS_OPT_R1_EPILOGUE in effect (0 log-
                           weights, no d^2 clamp; 1 clamp; 2 |d^2|; 3 none)  */
} ks_info;

/* Create a context for dimension K (1 <= K <= 4096) and bandwidth h (finite,
 * > 0, with log2(e)/(2h^2) finite in FP32), bound to the current CUDA device.
 * The default stream is the legacy default stream (0).
 * Errors: KS_EINVAL (K, h, out == NULL), KS_ECUDA / KS_EUNSUPPORTED (no
 * device, or device is not compute capability 10.0), KS_ENOMEM. */
KS_API ks_status ks_create(int K, float h, ks_ctx **out);

/* Destroy a context and free every library-owned buffer.  Synchronises the
 * context's stream first.  NULL is a no-op returning KS_OK. */
KS_API ks_status ks_destroy(ks_ctx *ctx);

/* Select the arithmetic (default KS_PREC_AUTO).  Takes effect at the next
 * ks_set_sources.  KS_EINVAL for an unknown value. */
KS_API ks_status ks_set_precision(ks_ctx *ctx, ks_precision p);

/* Set the CUDA stream (a cudaStream_t, passed as void*) every later call is
 * ordered on.  NULL means the legacy default stream. */
KS_API ks_status ks_set_stream(ks_ctx *ctx, void *cuda_stream);

/* Source preparation (Alg.1 l.3 vec_alpha; Eq.3):
 * copies alpha [M][K] and W [M][R] (DEVICE pointers, FP32, row-major) into
 * library-owned buffers: centred on the source mean, squared norms with FP64
 * accumulation, prescaled / split for the selected path, padded.
 * Stream-ordered: the caller keeps alpha and W alive and unmodified until the
 * stream passes this call.  Replaces any previous sources.
 * Errors: KS_EINVAL (M < 0, R < 1, R > 256, NULL with M > 0),
 * KS_EUNSUPPORTED (explicit FP32 precision with K > 32 or R > 1),
 * KS_ENOMEM, KS_ECUDA.  M == 0 is valid (every V becomes 0). */
KS_API ks_status ks_set_sources(ks_ctx *ctx, const float *alpha, const float *W,
                         int64_t M, int R);

/* Evaluate V [N][R] (DEVICE pointer, FP32, row-major) for targets beta [N][K]
 * (DEVICE pointer): one fused kernel launch (Alg.2) plus, when
 * the persistent schedule splits a target tile, an in-kernel deterministic
 * fix-up (no separate launch, no atomics on V).  Asynchronous on the
 * context's stream; V is OVERWRITTEN (not accumulated).  beta and V must not
 * overlap.  N == 0 is a no-op.  Library scratch grows on demand (a
 * synchronising allocation the first time a larger N is seen).
 * Errors: KS_ESTATE (no sources), KS_EINVAL (N < 0, NULL with N > 0),
 * KS_ENOMEM, KS_ECUDA. */
KS_API ks_status ks_eval(ks_ctx *ctx, const float *beta, int64_t N, float *V);

/* Same as ks_set_sources / ks_eval but alpha, W, beta, V are HOST pointers.
 * The library stages them through its own device buffers.  ks_set_sources_host
 * returns once alpha and W have been copied (the caller may reuse them); the
 * source preparation then runs on the context's stream.  ks_eval_host uploads
 * beta on a library copy stream (overlapping that preparation) in up to 4 chunks
 * for large N -- by default, for N >= 2 waves of 128-target tiles, a first chunk
 * of exactly one wave and the rest in one (KS_OPT_EVAL_CHUNK0 / _CHUNKS) --
 * evaluating chunk c while chunk c + 1 uploads and downloading its V while
 * chunk c + 1 evaluates, and returns after V is in host memory.  Pinned host
 * memory gives the fastest copies; pageable memory works.
 * ks_set_sources (device or host variant) may launch its statistics and
 * preparation as one cooperative kernel (KS_OPT_COOP_PREP); when the grid does
 * not fit the SMs available it falls back to separate kernels by itself. */
KS_API ks_status ks_set_sources_host(ks_ctx *ctx, const float *alpha, const float *W,
                              int64_t M, int R);
KS_API ks_status ks_eval_host(ks_ctx *ctx, const float *beta, int64_t N, float *V);

/* Tuning options.  Each selects among kernel variants that compute the same result
 * within the path's tolerance (SS3-SS4); none drops work.  Defaults are the
 * measured choices (SS7).  [sources] options take effect at the next
 * ks_set_sources, [eval] ones at the next ks_eval.  The environment variable named
 * beside an option, when set at ks_create, gives its initial value (read once there;
 * later calls never read the environment). */
typedef enum {
  KS_OPT_R1_KERNEL = 1,       /* KS_R1: 1 (default) the dedicated folded kernels where they apply
                                 (split-FP16, K <= 58: R = 1 and R > 1), 0 the general tcgen05
                                 kernel [sources] */
  KS_OPT_R1_EPILOGUE = 2,     /* KS_R1_MODE: 0 (default) log-weights when every W_i >= 0 (no
                                 d^2 >= 0 clamp; any W_i < 0 takes mode 1), 1 weights with the
                                 d^2 >= 0 clamp, 2 weights with d^2 -> |d^2|, 3 weights without
                                 a clamp [sources] */
  KS_OPT_EXP_POLY = 3,        /* KS_R1_POLY: exponential pairs of every 16 computed on the FMA
                                 pipe instead of MUFU (0, 4..8; -1 default) [eval] */
  KS_OPT_WEIGHTED_SUM = 4,    /* KS_TC_VCC: -1 auto, 0 tensor cores, 1 CUDA cores (R <= 16; the
                                 general kernel) [sources] */
  KS_OPT_LOG_WEIGHTS = 5,     /* KS_TC_LOGW: general kernel, R = 1: 1 (default) / 0 [sources] */
  KS_OPT_FOLD = 6,            /* KS_TC_FOLD: general kernel, R = 1: -1 auto, 0 off, 1 forced [sources] */
  KS_OPT_AUG = 7,             /* KS_TC_AUG: TF32 modes: -1 auto, 0, 1 norms in 2 K columns [sources] */
  KS_OPT_CLAMP = 8,           /* KS_TC_CLAMP: general kernel's log-weight epilogue: 0 (default),
                                 1 exact d^2 >= 0 clamp [eval] */
  KS_OPT_TARGET_RESIDENT = 9, /* KS_TC_ARES: general kernel: 1 (default) / 0 [eval] */
  KS_OPT_STAGES = 10,         /* KS_TC_STAGES: general kernel operand ring: 0 default, 3..5 [eval] */
  KS_OPT_AR_STAGES = 11,      /* KS_TC_AR_STAGES: 4 (default) / 5 [eval] */
  KS_OPT_WSLOTS = 12,         /* KS_TC_WSLOTS: 0 default, 2..4 [eval] */
  KS_OPT_PREP_LANES = 13,     /* KS_PREP_G: lanes per point in the prep kernels: 0 auto, 4, 8,
                                 16, 32 [sources, eval] */
  KS_OPT_EVAL_CHUNKS = 14,    /* KS_EVAL_CHUNKS: ks_eval_host target chunks: 0 auto, 1..4 [eval] */
  KS_OPT_FP32_SPLIT = 15,     /* KS_FP32_SPLIT: FP32 kernel tile body: -1 auto, 0, 1 [eval] */
  KS_OPT_MEASURE_CLOCK = 16,  /* 1: the R = 1 kernel records globaltimer and clock64 at every CTA's
                                 start and end, for ks_clock_read (measurement, 0 default) [eval] */
  KS_OPT_EVAL_CHUNK0 = 17,    /* KS_EVAL_CHUNK0: ks_eval_host first chunk in 128-target tiles: 0
                                 auto (one wave of tiles when N >= 2 waves), -1 equal chunks,
                                 t > 0 that many tiles [eval] */
  KS_OPT_COOP_PREP = 18,      /* KS_COOP_PREP: folded layouts (R = 1 and multi-column kernels):
                                 1 (default) source statistics and prep in one cooperative
                                 launch, 0 the separate kernels [sources] */
  KS_OPT_NARROW_PLANES = 19,  /* KS_NARROW_PLANES: R = 1 kernel: 1 (default) operand planes with
                                 only 16 used columns load as 32-byte rows -- the folded norm
                                 pieces at 27 <= K <= 32, the lo plane at 11 <= K <= 16 -- 0 as
                                 64-byte chunks [eval] */
  KS_OPT_COUNT_ = 20
} ks_option;

/* Set / read a tuning option.  KS_EINVAL for an unknown option or a value out of its range. */
KS_API ks_status ks_set_option(ks_ctx *ctx, ks_option opt, int value);
KS_API ks_status ks_get_option(const ks_ctx *ctx, ks_option opt, int *value);

/* Pre-size the scratch for targets up to N_max so later ks_eval calls never
 * allocate (useful before CUDA-graph capture).  KS_EINVAL if N_max < 0. */
KS_API ks_status ks_reserve(ks_ctx *ctx, int64_t N_max);

/* Report the configured path (see ks_info).  KS_EINVAL on NULL. */
KS_API ks_status ks_get_info(const ks_ctx *ctx, ks_info *out);

/* Kernel timing for the roofline report: when enabled, every fused-kernel
 * launch is bracketed by CUDA events on the launching stream.
 * ks_timing_read synchronises the stream and returns the summed device time
 * (ms) and number of timed launches since the last reset. */
KS_API ks_status ks_timing_enable(ks_ctx *ctx, int on);
KS_API ks_status ks_timing_read(ks_ctx *ctx, double *total_ms, int64_t *launches, int reset);

/* Effective SM clock of the last fused launch (KS_OPT_MEASURE_CLOCK = 1, R = 1 kernel): the mean
 * over its CTAs of elapsed SM cycles (clock64) / elapsed time (globaltimer), in GHz, and the CTA
 * count.  Synchronises the context's stream.  KS_ESTATE when no such launch was measured. */
KS_API ks_status ks_clock_read(ks_ctx *ctx, double *sm_ghz, int *ctas);

/* Human-readable status name; never NULL. */
KS_API const char *ks_status_str(ks_status s);

/* Thread-local detail of the last failing call on this thread ("" if none). */
KS_API const char *ks_last_error(void);

/* Library version string. */
KS_API const char *ks_version(void);

#ifdef __cplusplus
}
#endif

#endif /* KS_H_ */
