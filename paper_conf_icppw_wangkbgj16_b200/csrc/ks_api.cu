// ks_api.cu -- the C ABI of libks.so (include/ks.h): context, validation,
// library-owned buffers, path dispatch, stream-K launch configuration.
//
// Boundary passages: Eq.2 defines the inputs (sources
// alpha_i, weights W_i, targets beta_j, bandwidth h) and the output V; Alg.1
// lists A (M x K), B (K x N), W and V; A row-major / B
// column-major means one point's K coordinates are contiguous, which
// is the [points][K] layout taken here.
#include <cuda.h>
#include <cuda_runtime.h>

#include <cfloat>
#include <algorithm>
#include <cstdarg>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <new>
#include <string>
#include <vector>

#include "../../include/ks.h"
#include "ks_internal.h"
#include <nvtx3/nvToolsExt.h>

#ifndef KS_DEBUG
#define KS_DEBUG 0
#endif

namespace {

thread_local std::string g_err;

ks_status fail(ks_status s, const char* fmt, ...) __attribute__((format(printf, 2, 3)));
ks_status fail(ks_status s, const char* fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  g_err = buf;
  return s;
}

ks_status cuda_fail(cudaError_t e, const char* what) {
  return fail(e == cudaErrorMemoryAllocation ? KS_ENOMEM : KS_ECUDA, "%s: %s (%s)", what, cudaGetErrorName(e),
              cudaGetErrorString(e));
}

#define KS_CUDA(call, what)                      \
  do {                                           \
    cudaError_t e_ = (call);                     \
    if (e_ != cudaSuccess) return cuda_fail(e_, what); \
  } while (0)

typedef CUresult (*PFN_encodeTiled)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                    const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                    CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

PFN_encodeTiled get_encode() {
  static PFN_encodeTiled fn = nullptr;
  if (!fn) {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<PFN_encodeTiled>(p);
  }
  return fn;
}

int64_t round_up(int64_t x, int64_t m) { return (x + m - 1) / m * m; }

// Device buffer that grows on demand.  Growth synchronises the stream first
// (the old buffer may still be read by queued kernels).
template <typename T>
struct DBuf {
  T* p = nullptr;
  size_t cap = 0;  // elements
  cudaError_t reserve(size_t n, cudaStream_t st, bool zero) {
    if (n <= cap) return cudaSuccess;
    cudaError_t e = cudaStreamSynchronize(st);
    if (e != cudaSuccess) return e;
    if (p) cudaFree(p);
    p = nullptr;
    cap = 0;
    e = cudaMalloc(&p, n * sizeof(T));
    if (e != cudaSuccess) {
      p = nullptr;
      return e;
    }
    cap = n;
    if (zero) {
      e = cudaMemsetAsync(p, 0, n * sizeof(T), st);
      if (e != cudaSuccess) return e;
    }
    return cudaSuccess;
  }
  void release() {
    if (p) cudaFree(p);
    p = nullptr;
    cap = 0;
  }
};

}  // namespace

struct ks_ctx {
  int device = 0;
  int num_sms = 0;
  int K = 0;
  float h = 0.f;
  double c = 0.0;  // log2(e) / (2 h^2)
  ks_precision prec_req = KS_PREC_AUTO;
  cudaStream_t stream = nullptr;
  // host API: a copy stream for the target upload (overlaps the source prep still running on
  // `stream`) and events that end the host calls once their uploads are done
  cudaStream_t copy_stream = nullptr;
  cudaEvent_t ev_copied = nullptr;
  cudaEvent_t ev_bc[4] = {}, ev_v[4] = {};  // chunked ks_eval_host: chunk uploaded / evaluated
  cudaEvent_t ev_stream = nullptr;          // ks_set_stream: new stream waits for the old one
  int64_t reserve_n = 0;                    // ks_reserve: target count the scratch is sized for

  // current sources
  bool have_src = false;
  int path = KS_PATH_NONE;
  int prec_eff = KS_PREC_AUTO;
  int k_pad = 0;
  int64_t M = 0, m_pad = 0;
  int R = 1;
  DBuf<float> src;        // FP32 path: [k_pad + 2][m_pad]
  // TC path (tcgen05): TF32 hi/lo operand splits, norms, W^T splits
  DBuf<float> src_hi, src_lo, na, wt_hi, wt_lo, wv;
  DBuf<float> tgt_hi, tgt_lo, nb, tsc;   // FP16 mode: the hi/lo buffers hold halves
  DBuf<unsigned> amax;                   // FP16 mode: max |alpha - mu| (FP32 bits)
  DBuf<unsigned> wstat;                  // R = 1: {max |W| bits, any W < 0} (log-weight epilogue)
  bool tc_wstat = false;
  int tc_f16 = 0;
  int r_pad = 16;
  int tc_aug = 0;  // norms folded into the contraction as 2 extra K columns
  int tc_fold = 0;  // FP16 R = 1 folded layout (6 extra hi-plane K columns)
  int tc_kcols = 0, tc_kdims = 0;  // live operand columns / columns needing every split product
  int tc_vcc = 0;  // RV: weighted sum on CUDA cores over RV padded columns (0: tensor-core V path)
  int r1 = 0;      // R = 1 folded kernel (ks_fused_r1.cu): 2 = log-weight mode allowed, 3 = weight mode only
  int rv = 0;      // R > 1 folded kernel (ks_fused_rv.cu)
  int r1_clamp = 0;
  CUtensorMap tmB_hi, tmB_lo;
  CUtensorMap tmB_f;  // R = 1 narrow planes: the source hi plane's columns 32..47 (fold_narrow) or the lo
                      // plane's columns 0..15 (lo_narrow) as 32-byte boxes
  DBuf<float> mu;         // [k_pad]
  DBuf<double> mean_part; // [nparts][K]
  DBuf<float> mean_pmm;   // [nparts][K][2] column min/max
  DBuf<unsigned> mean_pw; // [nparts][2] weight statistics
  DBuf<unsigned> stats_counter;  // arrival counter of the statistics kernels (left zero)
  DBuf<unsigned> coop_bar;       // grid barrier of the cooperative source prep {arrivals, departures}
  DBuf<unsigned> wcol, wcol_part; // FP16 V-MMA: per-column max |W| bits [r_pad], block partials
  CUtensorMap tmap_src;

  // KS_OPT_MEASURE_CLOCK: per-CTA {globaltimer, clock64} x {start, end} of the last R = 1 launch
  DBuf<unsigned long long> clk_buf;
  int clk_ctas = 0;

  // eval scratch
  DBuf<float> partial;
  DBuf<int> counters;
  DBuf<unsigned long long> dbg_times;
  int last_grid = 0;

  // host staging (ks_*_host)
  DBuf<float> h_alpha, h_W, h_beta, h_V;

  // tuning options (ks_set_option; initial values from the environment at ks_create) and the
  // debug trace file (KS_CTA_TIMES, read at ks_create)
  ks::Opts opts;
  std::string cta_times_path;

  // accounting / timing
  int64_t launches = 0, fused_launches = 0;
  bool timing = false;
  std::vector<cudaEvent_t> ev;  // pairs (start, stop)
  size_t ev_used = 0;           // pairs in use
};

namespace ks {
thread_local const Opts* tl_opts = nullptr;
}

namespace {

// The context's options are visible to the launchers for the duration of one API call.
struct OptScope {
  const ks::Opts* prev;
  explicit OptScope(const ks_ctx* ctx) : prev(ks::tl_opts) { ks::tl_opts = &ctx->opts; }
  ~OptScope() { ks::tl_opts = prev; }
};

struct OptSpec {
  const char* env;
  int dflt, lo, hi;
};
// [option id] = {environment variable, default, valid range}
const OptSpec kOpt[KS_OPT_COUNT_] = {
    {nullptr, 0, 0, 0},
    {"KS_R1", 1, 0, 1},
    {"KS_R1_MODE", 0, 0, 3},
    {"KS_R1_POLY", -1, -1, 8},
    {"KS_TC_VCC", -1, -1, 1},
    {"KS_TC_LOGW", 1, 0, 1},
    {"KS_TC_FOLD", -1, -1, 1},
    {"KS_TC_AUG", -1, -1, 1},
    {"KS_TC_CLAMP", 0, 0, 1},
    {"KS_TC_ARES", 1, 0, 1},
    {"KS_TC_STAGES", 0, 0, 5},
    {"KS_TC_AR_STAGES", 4, 4, 5},
    {"KS_TC_WSLOTS", 0, 0, 4},
    {"KS_PREP_G", 0, 0, 32},
    {"KS_EVAL_CHUNKS", 0, 0, 4},
    {"KS_FP32_SPLIT", -1, -1, 1},
    {"KS_MEASURE_CLOCK", 0, 0, 1},
    {"KS_EVAL_CHUNK0", 0, -1, 1 << 20},
    {"KS_COOP_PREP", 1, 0, 1},
    {"KS_NARROW_PLANES", 1, 0, 1},
};

void init_opts(ks_ctx* ctx) {
  for (int i = 0; i < KS_OPT_COUNT_; ++i) {
    ctx->opts.v[i] = kOpt[i].dflt;
    if (!kOpt[i].env) continue;
    const char* e = getenv(kOpt[i].env);
    if (!e || !*e) continue;
    char* end = nullptr;
    const long v = strtol(e, &end, 10);
    if (end != e && v >= kOpt[i].lo && v <= kOpt[i].hi) ctx->opts.v[i] = (int)v;
  }
  const char* t = getenv("KS_CTA_TIMES");
  if (t && *t) ctx->cta_times_path = t;
}

ks_status check_ctx(const ks_ctx* ctx) {
  if (!ctx) return fail(KS_EINVAL, "ctx is NULL");
  return KS_OK;
}

ks_status set_device(const ks_ctx* ctx) {
  int cur = -1;
  KS_CUDA(cudaGetDevice(&cur), "cudaGetDevice");
  if (cur != ctx->device) KS_CUDA(cudaSetDevice(ctx->device), "cudaSetDevice");
  return KS_OK;
}

int fp32_k_pad(int K) { return K <= 4 ? 4 : K <= 8 ? 8 : K <= 16 ? 16 : 32; }

ks_status timed_begin(ks_ctx* ctx, cudaEvent_t* stop_out) {
  *stop_out = nullptr;
  if (!ctx->timing) return KS_OK;
  if (2 * ctx->ev_used + 2 > ctx->ev.size()) {
    cudaEvent_t a, b;
    KS_CUDA(cudaEventCreate(&a), "cudaEventCreate");
    KS_CUDA(cudaEventCreate(&b), "cudaEventCreate");
    ctx->ev.push_back(a);
    ctx->ev.push_back(b);
  }
  cudaEvent_t start = ctx->ev[2 * ctx->ev_used];
  *stop_out = ctx->ev[2 * ctx->ev_used + 1];
  KS_CUDA(cudaEventRecord(start, ctx->stream), "cudaEventRecord");
  return KS_OK;
}

ks_status timed_end(ks_ctx* ctx, cudaEvent_t stop) {
  if (!stop) return KS_OK;
  KS_CUDA(cudaEventRecord(stop, ctx->stream), "cudaEventRecord");
  ctx->ev_used++;
  return KS_OK;
}

// One launch: mu (always), amax (FP16 modes), wstat (want_w, R = 1).
cudaError_t source_stats(ks_ctx* ctx, const float* alpha, const float* W, bool want_w, int64_t M, int k_pad,
                         bool want_amax) {
  cudaStream_t st = ctx->stream;
  const int K = ctx->K;
  // ~2K coordinates per block (64 rows at K = 32, 8 rows at K = 256): one round of unrolled loads
  // per thread (the kernel is load-latency bound); beyond 256 blocks the partials are reduced by
  // K + 1 blocks (launch_source_stats), not the last block alone
  const int64_t rows = K >= 2048 ? 1 : 2048 / K;
  int64_t np64 = (M + rows - 1) / rows;
  if (np64 < 1) np64 = 1;
  if (np64 > 4096) np64 = 4096;
  const int nparts = (int)np64;
  cudaError_t e;
  if ((e = ctx->mean_part.reserve((size_t)nparts * K, st, false)) != cudaSuccess) return e;
  if ((e = ctx->mean_pmm.reserve((size_t)nparts * K * 2, st, false)) != cudaSuccess) return e;
  if ((e = ctx->mean_pw.reserve((size_t)nparts * 2, st, false)) != cudaSuccess) return e;
  if ((e = ctx->stats_counter.reserve(1, st, true)) != cudaSuccess) return e;
  if ((e = ctx->mu.reserve(k_pad, st, false)) != cudaSuccess) return e;
  if (want_amax && (e = ctx->amax.reserve(1, st, false)) != cudaSuccess) return e;
  if (want_w && (e = ctx->wstat.reserve(2, st, false)) != cudaSuccess) return e;
  ctx->launches += (K > 32 || nparts > 256) ? 2 : 1;  // launch_source_stats' split
  return ks::launch_source_stats(alpha, W, M, K, k_pad, nparts, ctx->mean_part.p, ctx->mean_pmm.p, ctx->mean_pw.p,
                                 ctx->stats_counter.p, ctx->mu.p, want_amax ? ctx->amax.p : nullptr,
                                 want_w ? ctx->wstat.p : nullptr, st);
}

ks_status prepare_fp32(ks_ctx* ctx, const float* alpha, const float* W, int64_t M) {
  const int K = ctx->K;
  const int k_pad = fp32_k_pad(K);
  const int64_t m_pad = round_up(M > 0 ? M : 1, ks::kTileS);
  cudaStream_t st = ctx->stream;
  const size_t need = (size_t)(k_pad + 2) * (size_t)m_pad;
  KS_CUDA(ctx->src.reserve(need, st, false), "allocate source buffer");
  KS_CUDA(ctx->mu.reserve(k_pad, st, false), "allocate mean buffer");
  KS_CUDA(source_stats(ctx, alpha, nullptr, false, M, k_pad, false), "source mean");
  KS_CUDA(ks::launch_prep_fp32(alpha, W, M, m_pad, K, k_pad, ctx->mu.p, ctx->c, ctx->src.p, st), "source prep");
  ctx->launches += 1;

  PFN_encodeTiled enc = get_encode();
  if (!enc) return fail(KS_ECUDA, "cuTensorMapEncodeTiled unavailable from the driver");
  cuuint64_t dims[2] = {(cuuint64_t)m_pad, (cuuint64_t)(k_pad + 2)};
  cuuint64_t strides[1] = {(cuuint64_t)m_pad * sizeof(float)};
  cuuint32_t box[2] = {(cuuint32_t)ks::kTileS, (cuuint32_t)(k_pad + 2)};
  cuuint32_t estr[2] = {1, 1};
  CUresult r = enc(&ctx->tmap_src, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, ctx->src.p, dims, strides, box, estr,
                   CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return fail(KS_ECUDA, "cuTensorMapEncodeTiled failed (CUresult %d)", (int)r);

  ctx->k_pad = k_pad;
  ctx->m_pad = m_pad;
  return KS_OK;
}

ks_status eval_fp32(ks_ctx* ctx, const float* beta, int64_t N, float* V) {
  cudaStream_t st = ctx->stream;
  ks::StreamK sk;
  sk.n_t = (N + ks::kTileT - 1) / ks::kTileT;
  sk.n_s = (int32_t)(ctx->m_pad / ks::kTileS);
  sk.units = sk.n_t * (int64_t)sk.n_s;
  int64_t g = (int64_t)ctx->num_sms * ks::fused_fp32_ctas_per_sm(ctx->k_pad);
  if (g > sk.units) g = sk.units;  // every CTA owns >= 1 unit (fix-up relies on it)
  sk.grid = (int32_t)g;
  KS_CUDA(ctx->partial.reserve((size_t)sk.grid * 2 * ks::kTileT, st, false), "allocate partials");
  KS_CUDA(ctx->counters.reserve((size_t)sk.n_t, st, true), "allocate tile counters");

  ks::Fp32Args a;
  a.beta = beta;
  a.N = N;
  a.K = ctx->K;
  a.mu = ctx->mu.p;
  a.c = ctx->c;
  a.V = V;
  a.partial = ctx->partial.p;
  a.counters = ctx->counters.p;
  a.sk = sk;
  a.cta_times = nullptr;
  // debug trace: KS_CTA_TIMES=<file> (at ks_create) appends per-CTA start/end globaltimer (ns)
  const char* dbg = ctx->cta_times_path.empty() ? nullptr : ctx->cta_times_path.c_str();
  if (dbg) {
    KS_CUDA(ctx->dbg_times.reserve((size_t)sk.grid * 2, st, true), "allocate debug timers");
    a.cta_times = ctx->dbg_times.p;
  }
  cudaEvent_t stop;
  ks_status s = timed_begin(ctx, &stop);
  if (s != KS_OK) return s;
  KS_CUDA(ks::launch_fused_fp32(&ctx->tmap_src, ctx->k_pad, a, st), "fused FP32 kernel launch");
  ctx->launches++;
  ctx->fused_launches++;
  ctx->last_grid = sk.grid;
  ks_status ts = timed_end(ctx, stop);
  if (a.cta_times) {
    std::vector<unsigned long long> h((size_t)sk.grid * 2);
    KS_CUDA(cudaMemcpyAsync(h.data(), a.cta_times, h.size() * 8, cudaMemcpyDeviceToHost, st), "copy debug timers");
    KS_CUDA(cudaStreamSynchronize(st), "synchronize");
    FILE* f = fopen(dbg, "a");
    if (f) {
      for (int i = 0; i < sk.grid; ++i) fprintf(f, "%d %llu %llu\n", i, h[2 * i], h[2 * i + 1]);
      fprintf(f, "--\n");
      fclose(f);
    }
  }
  return ts;
}


// Row-major [rows][inner] operand, one box = box_rows x 64 bytes (16 FP32 or
// 32 FP16 elements), SWIZZLE_64B: the K-major smem layout of the MMA operands.
ks_status encode_2d_sw64(CUtensorMap* map, const void* base, int64_t inner, int64_t rows, int box_rows,
                         bool f16 = false, bool rows32 = false) {
  PFN_encodeTiled enc = get_encode();
  if (!enc) return fail(KS_ECUDA, "cuTensorMapEncodeTiled unavailable from the driver");
  const size_t es = f16 ? 2 : 4;
  const size_t row_bytes = rows32 ? 32 : 64;  // rows32: 32-byte boxes with SWIZZLE_32B
  cuuint64_t dims[2] = {(cuuint64_t)inner, (cuuint64_t)rows};
  cuuint64_t strides[1] = {(cuuint64_t)inner * es};
  cuuint32_t box[2] = {(cuuint32_t)(row_bytes / es), (cuuint32_t)box_rows};
  cuuint32_t estr[2] = {1, 1};
  CUresult r = enc(map, f16 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2,
                   const_cast<void*>(base), dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                   rows32 ? CU_TENSOR_MAP_SWIZZLE_32B : CU_TENSOR_MAP_SWIZZLE_64B,
                   CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return fail(KS_ECUDA, "cuTensorMapEncodeTiled (2D SW64) failed (CUresult %d)", (int)r);
  return KS_OK;
}

// W^T [r_pad][m_pad] viewed as {16 sources, r, m_pad/16 chunks}: one box =
// 8 chunks x r_c rows x 16 floats = the K-major SWIZZLE_64B B operand of V-MMA.
ks_status encode_wt(CUtensorMap* map, const float* base, int64_t m_pad, int r_pad, int r_c) {
  PFN_encodeTiled enc = get_encode();
  if (!enc) return fail(KS_ECUDA, "cuTensorMapEncodeTiled unavailable from the driver");
  cuuint64_t dims[3] = {16, (cuuint64_t)r_pad, (cuuint64_t)(m_pad / 16)};
  cuuint64_t strides[2] = {(cuuint64_t)m_pad * sizeof(float), 64};
  cuuint32_t box[3] = {16, (cuuint32_t)r_c, (cuuint32_t)(ks::kTcTileS / 16)};
  cuuint32_t estr[3] = {1, 1, 1};
  CUresult r = enc(map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3, const_cast<float*>(base), dims, strides, box, estr,
                   CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_64B, CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return fail(KS_ECUDA, "cuTensorMapEncodeTiled (W^T 3D) failed (CUresult %d)", (int)r);
  return KS_OK;
}

// wcat [2 r_pad][m_pad] FP16 viewed as {32 sources, 2 r_pad rows, m_pad/32 chunks}: one box =
// 4 chunks x 2 r_c rows x 64 B = the K-major SWIZZLE_64B B operand ([W_hi | W_lo] rows) of the
// FP16 V-MMA for one 128-source tile.
ks_status encode_wcat(CUtensorMap* map, const void* base, int64_t m_pad, int r_pad, int r_c, int tile_s) {
  PFN_encodeTiled enc = get_encode();
  if (!enc) return fail(KS_ECUDA, "cuTensorMapEncodeTiled unavailable from the driver");
  cuuint64_t dims[3] = {32, (cuuint64_t)(2 * r_pad), (cuuint64_t)(m_pad / 32)};
  cuuint64_t strides[2] = {(cuuint64_t)m_pad * 2, 64};
  cuuint32_t box[3] = {32, (cuuint32_t)(2 * r_c), (cuuint32_t)(tile_s / 32)};
  cuuint32_t estr[3] = {1, 1, 1};
  CUresult r = enc(map, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 3, const_cast<void*>(base), dims, strides, box, estr,
                   CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_64B, CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return fail(KS_ECUDA, "cuTensorMapEncodeTiled (wcat 3D) failed (CUresult %d)", (int)r);
  return KS_OK;
}

// Fold the norms into the MMA (two extra K columns) when that costs no extra K chunk.
// KS_TC_AUG=0/1 overrides (measurement knob).
int tc_aug(int K) {
  const int o = ks::opt(KS_OPT_AUG, -1);
  if (o == 0 || o == 1) return o;
  return (round_up(K + 2, ks::kTcKC) == round_up(K, ks::kTcKC)) ? 1 : 0;  // measured: an extra chunk costs more than it saves
}
int tc_k_pad(int K) { return (int)round_up(K + 2 * tc_aug(K), ks::kTcKC); }

ks_status prepare_tc(ks_ctx* ctx, const float* alpha, const float* W, int64_t M, int R) {
  const int K = ctx->K;
  const bool f16 = ctx->prec_eff == KS_PREC_3XF16;
  // Weighted sum: on CUDA cores (vcc = padded R, 256-source tiles) or as a second tensor-core
  // MMA (vcc = 0).  Split-FP16 crossover measured at M = N = 65,536 (tools/vsweep.py, DESIGN.md
  // SS7): the tensor-core V costs the same for any R, the CUDA-core V grows with R -- CUDA cores
  // for R <= 4, for R <= 8 when K > 48, and for R <= 16 when K >= 256 (measured round 2,
  // profiles/r02/policy_sweeps.txt: K = 256, R = 16 at 262,144^2 ties within 0.5%, R = 8 is 20%
  // faster on CUDA cores); TF32 modes keep CUDA cores up to R = 16.
  // KS_OPT_WEIGHTED_SUM = 0 / 1 forces the tensor-core / CUDA-core (R <= 16) variant.
  const int ovs = ks::opt(KS_OPT_WEIGHTED_SUM, -1);
  int vcc = ks::fused_tc_rv(R);
  if (f16 && (R > 8 || (R > 4 && K <= 48)) && !(K >= 256 && R <= 16)) vcc = 0;
  if (ovs == 0) vcc = 0;
  if (ovs == 1) vcc = ks::fused_tc_rv(R);
  // R = 1 with W >= 0: log-weights in na (decided on the device, no host sync);
  // KS_OPT_LOG_WEIGHTS = 0 disables (general kernel)
  const bool use_wstat = (vcc == 1) && ks::opt(KS_OPT_LOG_WEIGHTS, 1) != 0;
  // FP16, R = 1: folded layout (norms + log-weights as 6 extra hi-plane K columns, reading
  // Q26; active on the device when c K amax^2 <= 2^12).  KS_TC_FOLD=0 disables (measurement knob)
  // Measured (tools/fsweep.py, profiles/r01/policy_sweeps.txt): the fold pays up to K = 48 even
  // when its columns need an operand chunk of their own, and costs ~1-4% beyond that when they do
  // (K = 64, 96, 128, ...) -- then the norms stay in the epilogue.
  const int ofo = ks::opt(KS_OPT_FOLD, -1);
  const bool fold_fits = K <= 48 || round_up(K + 6, 2 * ks::kTcKC) == round_up(K, 2 * ks::kTcKC);
  int fold = (f16 && use_wstat && ofo != 0 && (fold_fits || ofo == 1)) ? 1 : 0;
  // R = 1, split-FP16, K + 6 <= 64: the dedicated folded kernel (ks_fused_r1.cu;
  // KS_OPT_R1_KERNEL = 0 selects the general kernel), fold mode 2 (always folded, fold shift,
  // reading Q28).  KS_OPT_R1_EPILOGUE: 0 = log-weights when every W_i >= 0 (decided on the
  // device), else the weight mode with the clamp; 1 = weight mode with the d^2 >= 0 clamp for any
  // W; 2 = weight mode with |d^2|; 3 = weight mode without a clamp.
  int r1 = 0, r1_clamp = 0, rv = 0;
  if (f16 && vcc == 1 && K + 6 <= 2 * 2 * ks::kTcKC && ks::opt(KS_OPT_R1_KERNEL, 1) != 0) {
    const int mode = ks::opt(KS_OPT_R1_EPILOGUE, 0);
    r1 = mode == 0 ? 2 : 3;
    r1_clamp = mode == 3 ? 0 : mode == 2 ? 2 : 1;
    fold = r1;
  }
  // R > 1, split-FP16, K + 6 <= 64: the multi-column kernel (ks_fused_rv.cu) on the same skeleton,
  // weighted sum as a second tcgen05 MMA (fold mode 3: the norms in the contraction with the fold
  // shift, no log-weights; the FP16 weight split of reading Q27).  KS_OPT_R1_KERNEL = 0 selects
  // the general kernel for both.
  if (f16 && R > 1 && K + 6 <= 2 * 2 * ks::kTcKC && ks::opt(KS_OPT_R1_KERNEL, 1) != 0 &&
      ks::opt(KS_OPT_WEIGHTED_SUM, -1) != 1) {
    rv = 1;
    vcc = 0;
    fold = 3;
  }
  // k_pad in elements: one 64-byte row chunk per pipeline stage = 16 FP32 or 32 FP16; the R = 1
  // kernel at K + 6 <= 16 keeps 32-byte rows (16 halves: half the operand bytes; cfg5's prepared
  // source set, 1,048,576 x 2 x 32 B, then stays in the 126 MB L2)
  const bool narrow = (r1 || rv) && K + 6 <= ks::kTcKC;
  const int k_pad = narrow ? ks::kTcKC
                    : f16 ? (int)round_up(K + 6 * (fold ? 1 : 0), 2 * ks::kTcKC) : tc_k_pad(K);
  const int aug = f16 ? 0 : tc_aug(K);  // FP16 mode: norms stay in FP32 in the epilogue (or fold)
  const int tile_s = ks::fused_tc_tile_s(vcc);
  const int box_s = r1 ? 128 : rv ? ks::kRvTileS : tile_s;  // sources per operand tile of the kernel
  const int64_t m_pad = round_up(M > 0 ? M : 1, rv ? ks::kRvTileS : tile_s);
  const int r_pad = (int)round_up(R, 16);
  cudaStream_t st = ctx->stream;
  const size_t nsrc = f16 ? ((size_t)m_pad * k_pad + 1) / 2 : (size_t)m_pad * k_pad, nw = (size_t)r_pad * m_pad;
  KS_CUDA(ctx->src_hi.reserve(nsrc, st, false), "allocate source hi");
  KS_CUDA(ctx->src_lo.reserve(nsrc, st, false), "allocate source lo");
  KS_CUDA(ctx->na.reserve((size_t)m_pad, st, false), "allocate source norms");
  KS_CUDA(ctx->wt_hi.reserve(nw, st, false), "allocate W hi");
  KS_CUDA(ctx->wt_lo.reserve(nw, st, false), "allocate W lo");
  KS_CUDA(ctx->wv.reserve((size_t)m_pad * (vcc ? vcc : 1), st, false), "allocate W rows");
  KS_CUDA(ctx->mu.reserve(k_pad, st, false), "allocate mean buffer");
  // mean, max |alpha - mu| (FP16 scaling) and the R = 1 weight statistics in one launch
  const bool want_wstat = use_wstat || r1;  // the R = 1 kernel decides its epilogue from wstat
  // folded layouts (the R = 1 and multi-column kernels): statistics and source prep in one
  // cooperative launch (KS_OPT_COOP_PREP = 0: the separate statistics and prep kernels)
  bool coop = f16 && fold >= 2 && K + 6 <= k_pad && (k_pad == 16 || k_pad == 32 || k_pad == 64) &&
              ks::opt(KS_OPT_PREP_LANES, 0) == 0 && ks::opt(KS_OPT_COOP_PREP, 1) != 0;
  if (coop) {
    const int grid = ks::coop_prep_grid(k_pad, m_pad, ctx->num_sms);
    KS_CUDA(ctx->mean_part.reserve((size_t)grid * K, st, false), "allocate statistics partials");
    KS_CUDA(ctx->mean_pmm.reserve((size_t)grid * K * 2, st, false), "allocate statistics partials");
    KS_CUDA(ctx->mean_pw.reserve((size_t)grid * 2, st, false), "allocate statistics partials");
    KS_CUDA(ctx->coop_bar.reserve(2, st, true), "allocate grid barrier");
    KS_CUDA(ctx->stats_counter.reserve(1, st, true), "allocate statistics counter");  // the W column prep
    KS_CUDA(ctx->amax.reserve(1, st, false), "allocate amax");
    if (want_wstat) KS_CUDA(ctx->wstat.reserve(2, st, false), "allocate weight statistics");
    const cudaError_t ce = ks::launch_prep_fold_sources_coop(
        alpha, W, M, m_pad, K, k_pad, R, ctx->c, fold, grid, ctx->mean_part.p, ctx->mean_pmm.p, ctx->mean_pw.p,
        ctx->coop_bar.p, ctx->mu.p, ctx->amax.p, want_wstat ? ctx->wstat.p : nullptr, ctx->src_hi.p, ctx->src_lo.p,
        ctx->na.p, ctx->wv.p, vcc, st);
    if (ce == cudaErrorCooperativeLaunchTooLarge) {  // fewer SMs than the device reports (MPS, partitions):
      (void)cudaGetLastError();                       // the separate statistics and prep kernels instead
      coop = false;
    } else {
      KS_CUDA(ce, "statistics + source prep (cooperative, folded)");
    }
  }
  if (!coop) KS_CUDA(source_stats(ctx, alpha, W, want_wstat, M, k_pad, f16), "source statistics");
  const unsigned* wst = want_wstat ? ctx->wstat.p : nullptr;
  if (f16) {
    if (!coop) {
      KS_CUDA(ks::launch_prep_f16_sources(alpha, W, M, m_pad, K, k_pad, R, 0, ctx->mu.p, ctx->c,
                                          ctx->amax.p, fold, ctx->src_hi.p, ctx->src_lo.p, ctx->na.p, ctx->wt_hi.p,
                                          ctx->wt_lo.p, ctx->wv.p, vcc, wst, st),
              "source prep (TC, FP16)");
    }
    if (vcc == 0) {  // weighted sum on the tensor cores in FP16 (reading Q27): wcat in the W hi buffer
      int np = (int)((M + 1023) / 1024);
      if (np < 1) np = 1;
      if (np > 256) np = 256;
      KS_CUDA(ctx->wcol.reserve((size_t)r_pad, st, true), "allocate W column scales");
      KS_CUDA(ctx->wcol_part.reserve((size_t)np * R, st, false), "allocate W column partials");
      KS_CUDA(ks::launch_prep_wcat(W, M, m_pad, R, r_pad, np, ctx->wcol_part.p, ctx->stats_counter.p, ctx->wcol.p,
                                   ctx->wt_hi.p, st),
              "weight prep (FP16 V-MMA)");
      ctx->launches += (M > 0) ? 2 : 1;
    }
  } else {
    KS_CUDA(ks::launch_prep_tc_sources(alpha, W, M, m_pad, K, k_pad, R, vcc ? 0 : r_pad, ctx->mu.p, ctx->c, aug,
                                       ctx->src_hi.p, ctx->src_lo.p, ctx->na.p, ctx->wt_hi.p, ctx->wt_lo.p,
                                       ctx->wv.p, vcc, wst, st),
            "source prep (TC)");
  }
  ctx->launches += 1;
  ks_status s = encode_2d_sw64(&ctx->tmB_hi, ctx->src_hi.p, k_pad, m_pad, box_s, f16, narrow);
  if (s != KS_OK) return s;
  s = encode_2d_sw64(&ctx->tmB_lo, ctx->src_lo.p, k_pad, m_pad, box_s, f16, narrow);
  if (s != KS_OK) return s;
  if (r1 && k_pad == 64) {  // the fold chunk as one 16-column plane (fold_narrow, eval_r1)
    s = encode_2d_sw64(&ctx->tmB_f, ctx->src_hi.p, k_pad, m_pad, box_s, true, true);
    if (s != KS_OK) return s;
  } else if (r1 && k_pad == 32 && K <= 16) {  // the lo plane as 16 columns (lo_narrow, eval_r1)
    s = encode_2d_sw64(&ctx->tmB_f, ctx->src_lo.p, k_pad, m_pad, box_s, true, true);
    if (s != KS_OK) return s;
  }
  ctx->k_pad = k_pad;
  ctx->m_pad = m_pad;
  ctx->r_pad = r_pad;
  ctx->tc_aug = aug;
  ctx->tc_fold = fold;  // 1: general kernel (device-side f16_fold_ok); 2, 3: R = 1 kernel (fold shift)
  ctx->r1 = r1;
  ctx->r1_clamp = r1_clamp;
  ctx->rv = rv;
  ctx->tc_kcols = f16 ? K + 6 * (fold ? 1 : 0) : K + 2 * aug;
  ctx->tc_kdims = f16 ? K : K + 2 * aug;
  ctx->tc_vcc = vcc;
  ctx->tc_f16 = f16 ? 1 : 0;
  ctx->tc_wstat = want_wstat;
  return KS_OK;
}

// R = 1 folded kernel (ks_fused_r1.cu): 128-source units, one launch.
ks_status eval_r1(ks_ctx* ctx, const CUtensorMap* maps, int64_t N, float* V) {
  cudaStream_t st = ctx->stream;
  ks::StreamK sk;
  sk.n_t = round_up(N, ks::kTcTileT) / ks::kTcTileT;
  sk.n_s = (int32_t)(ctx->m_pad / 128);
  sk.units = sk.n_t * (int64_t)sk.n_s;
  int64_t g = ctx->num_sms;
  if (g > sk.units) g = sk.units;
  sk.grid = (int32_t)g;
  KS_CUDA(ctx->partial.reserve((size_t)sk.grid * 2 * 128, st, false), "allocate partials");
  KS_CUDA(ctx->counters.reserve((size_t)sk.n_t, st, true), "allocate tile counters");
  ks::R1Args a;
  // the second operand chunk holds only the folded norm pieces: load it as one 16-column plane
  a.fold_narrow = (ctx->k_pad == 64 && ctx->tc_kdims <= 32 && ctx->tc_kcols <= 48 &&
                   ctx->opts.v[KS_OPT_NARROW_PLANES] != 0) ? 1 : 0;
  // one chunk with coordinates only in its first 16 columns: the lo plane as 16 columns
  a.lo_narrow = (ctx->k_pad == 32 && ctx->tc_kdims <= 16 && ctx->opts.v[KS_OPT_NARROW_PLANES] != 0) ? 1 : 0;
  a.N = N;
  a.narrow = ctx->k_pad == ks::kTcKC ? 1 : 0;
  a.n_kc = a.narrow ? 1 : ctx->k_pad / 32;
  a.kdims = ctx->tc_kdims;
  a.kcols = ctx->tc_kcols;
  a.logw = ctx->r1 == 2 ? 1 : 0;
  a.clamp = ctx->r1_clamp;
  a.wstat = ctx->wstat.p;
  a.wv = ctx->wv.p;
  a.V = V;
  a.partial = ctx->partial.p;
  a.counters = ctx->counters.p;
  a.sk = sk;
  a.cta_times = nullptr;
  a.dbg = 0;
#if KS_DEBUG
  {
    const char* e = getenv("KS_R1_DEBUG");  // measurement builds only: drops work, wrong results
    a.dbg = e ? atoi(e) : 0;
  }
#endif
  const char* dbg = ctx->cta_times_path.empty() ? nullptr : ctx->cta_times_path.c_str();
  const size_t n_dbg = (size_t)sk.grid * (4 + 20 * 4) + 4 * 4096;  // + KS_TRACE unit clocks of CTA 0
  if (dbg) {
    KS_CUDA(ctx->dbg_times.reserve(n_dbg, st, true), "allocate debug timers");
    a.cta_times = ctx->dbg_times.p;
  } else if (ctx->opts.v[KS_OPT_MEASURE_CLOCK]) {
    KS_CUDA(ctx->clk_buf.reserve((size_t)ctx->num_sms * 4, st, false), "allocate clock buffer");
    a.cta_times = ctx->clk_buf.p;
    ctx->clk_ctas = sk.grid;
  }
  cudaEvent_t stop;
  ks_status s = timed_begin(ctx, &stop);
  if (s != KS_OK) return s;
  KS_CUDA(ks::launch_fused_r1(maps, a, ks::r1_poly(), st), "fused R = 1 kernel launch");
  ctx->launches++;
  ctx->fused_launches++;
  ctx->last_grid = sk.grid;
  s = timed_end(ctx, stop);
  if (s != KS_OK) return s;
  if (dbg) {  // "r1 <cta> <t0 ns> <t1 ns> <clock0> <clock1> [20 x 4 phase clocks]" per CTA
    std::vector<unsigned long long> h(n_dbg);
    KS_CUDA(cudaMemcpyAsync(h.data(), a.cta_times, h.size() * 8, cudaMemcpyDeviceToHost, st), "copy debug timers");
    KS_CUDA(cudaStreamSynchronize(st), "synchronize");
    FILE* f = fopen(dbg, "a");
    if (f) {
      for (int i = 0; i < sk.grid; ++i) {
        fprintf(f, "r1 %d %llu %llu %llu %llu", i, h[4 * i], h[4 * i + 2], h[4 * i + 1], h[4 * i + 3]);
        for (int k = 0; k < 80; ++k) fprintf(f, " %llu", h[4 * (size_t)sk.grid + (size_t)i * 80 + k]);
        fprintf(f, "\n");
      }
      const size_t t0 = (size_t)sk.grid * 84;
      for (int q = 0; q < 4096 && h[t0 + 4 * q] != 0; ++q)
        fprintf(f, "trace %d %llu %llu %llu %llu\n", q, h[t0 + 4 * q], h[t0 + 4 * q + 1], h[t0 + 4 * q + 2],
                h[t0 + 4 * q + 3]);
      fprintf(f, "--\n");
      fclose(f);
    }
  }
  return KS_OK;
}

// R > 1 folded kernel (ks_fused_rv.cu): 96-source units, one launch per block of 16 or 32
// weight columns.
ks_status eval_rv(ks_ctx* ctx, CUtensorMap* maps, int64_t N, float* V) {
  cudaStream_t st = ctx->stream;
  ks::StreamK sk;
  sk.n_t = round_up(N, ks::kTcTileT) / ks::kTcTileT;
  sk.n_s = (int32_t)(ctx->m_pad / ks::kRvTileS);
  sk.units = sk.n_t * (int64_t)sk.n_s;
  int64_t g = ctx->num_sms;
  if (g > sk.units) g = sk.units;
  sk.grid = (int32_t)g;
  KS_CUDA(ctx->partial.reserve((size_t)sk.grid * 2 * 128 * 32, st, false), "allocate partials");
  KS_CUDA(ctx->counters.reserve((size_t)sk.n_t, st, true), "allocate tile counters");
  ks::RvArgs a;
  a.N = N;
  a.narrow = ctx->k_pad == ks::kTcKC ? 1 : 0;
  a.n_kc = a.narrow ? 1 : ctx->k_pad / 32;
  a.kdims = ctx->tc_kdims;
  a.kcols = ctx->tc_kcols;
  a.R = ctx->R;
  a.wcol = ctx->wcol.p;
  a.V = V;
  a.partial = ctx->partial.p;
  a.counters = ctx->counters.p;
  a.sk = sk;
  a.trace = nullptr;
  a.cta_times = nullptr;
  if (ctx->opts.v[KS_OPT_MEASURE_CLOCK]) {  // the first launch (columns 0 .. r_c - 1) is measured
    KS_CUDA(ctx->clk_buf.reserve((size_t)ctx->num_sms * 4, st, false), "allocate clock buffer");
    a.cta_times = ctx->clk_buf.p;
    ctx->clk_ctas = sk.grid;
  }
  a.dbg = 0;
#if KS_DEBUG
  {
    const char* e = getenv("KS_RV_DEBUG");  // measurement builds only: drops work, wrong results
    a.dbg = e ? atoi(e) : 0;
  }
#endif
  const char* dbg = ctx->cta_times_path.empty() ? nullptr : ctx->cta_times_path.c_str();
  if (dbg) {  // KS_TRACE builds write the unit clocks of CTA 0 (first 16/32-column launch)
    KS_CUDA(ctx->dbg_times.reserve((size_t)12 * 4096, st, true), "allocate debug timers");
    KS_CUDA(cudaMemsetAsync(ctx->dbg_times.p, 0, (size_t)12 * 4096 * 8, st), "zero debug timers");
    a.trace = ctx->dbg_times.p;
  }
  for (int r_off = 0; r_off < ctx->r_pad;) {
    const int r_c = (ctx->r_pad - r_off >= 32) ? 32 : 16;
    a.r_c = r_c;
    a.r_off = r_off;
    a.r_valid = (ctx->R - r_off < r_c) ? (ctx->R - r_off) : r_c;
    ks_status s = encode_wcat(&maps[4], ctx->wt_hi.p, ctx->m_pad, ctx->r_pad, r_c, ks::kRvTileS);
    if (s != KS_OK) return s;
    cudaEvent_t stop;
    s = timed_begin(ctx, &stop);
    if (s != KS_OK) return s;
    KS_CUDA(ks::launch_fused_rv(maps, a, st), "fused R > 1 kernel launch");
    ctx->launches++;
    ctx->fused_launches++;
    ctx->last_grid = sk.grid;
    s = timed_end(ctx, stop);
    if (s != KS_OK) return s;
    r_off += r_c;
    a.trace = nullptr;
    a.cta_times = nullptr;
  }
  if (dbg) {
    std::vector<unsigned long long> h((size_t)12 * 4096);
    KS_CUDA(cudaMemcpyAsync(h.data(), ctx->dbg_times.p, h.size() * 8, cudaMemcpyDeviceToHost, st), "copy trace");
    KS_CUDA(cudaStreamSynchronize(st), "synchronize");
    FILE* f = fopen(dbg, "a");
    if (f) {  // per unit: S issued, epilogue wake, P ready, V issued, S waits done, V waits done,
              // V vempty done, V pready done, fold start, fold end, -, -
      for (int q = 0; q < 4096 && h[12 * q] != 0; ++q) {
        fprintf(f, "trace %d", q);
        for (int k = 0; k < 12; ++k) fprintf(f, " %llu", h[12 * q + k]);
        fprintf(f, "\n");
      }
      fprintf(f, "--\n");
      fclose(f);
    }
  }
  return KS_OK;
}

ks_status eval_tc(ks_ctx* ctx, const float* beta, int64_t N, float* V) {
  cudaStream_t st = ctx->stream;
  const int k_pad = ctx->k_pad;
  const int64_t n_pad = round_up(N, ks::kTcTileT);
  const bool f16 = ctx->tc_f16 != 0;
  const size_t ntg = f16 ? ((size_t)n_pad * k_pad + 1) / 2 : (size_t)n_pad * k_pad;
  KS_CUDA(ctx->tgt_hi.reserve(ntg, st, false), "allocate target hi");
  KS_CUDA(ctx->tgt_lo.reserve(ntg, st, false), "allocate target lo");
  KS_CUDA(ctx->nb.reserve((size_t)n_pad, st, false), "allocate target norms");
  KS_CUDA(ctx->tsc.reserve((size_t)n_pad, st, false), "allocate target scales");
  if (f16) {
    KS_CUDA(ks::launch_prep_f16_targets(beta, N, n_pad, ctx->K, k_pad, ctx->mu.p, ctx->c, ctx->amax.p,
                                        ctx->tc_fold, ctx->tgt_hi.p, ctx->tgt_lo.p, ctx->nb.p, ctx->tsc.p, st),
            "target prep (TC, FP16)");
  } else {
    KS_CUDA(ks::launch_prep_tc_targets(beta, N, n_pad, ctx->K, k_pad, ctx->mu.p, ctx->c, ctx->tc_aug,
                                       ctx->tgt_hi.p, ctx->tgt_lo.p, ctx->nb.p, ctx->tsc.p, st),
            "target prep (TC)");
  }
  ctx->launches += 1;
  CUtensorMap maps[6];
  const bool narrow = (ctx->r1 || ctx->rv) && k_pad == ks::kTcKC;  // 32-byte operand rows (K + 6 <= 16)
  ks_status s = encode_2d_sw64(&maps[0], ctx->tgt_hi.p, k_pad, n_pad, ks::kTcTileT, f16, narrow);
  if (s != KS_OK) return s;
  s = encode_2d_sw64(&maps[1], ctx->tgt_lo.p, k_pad, n_pad, ks::kTcTileT, f16, narrow);
  if (s != KS_OK) return s;
  maps[2] = ctx->tmB_hi;
  maps[3] = ctx->tmB_lo;
  if (ctx->r1) {  // the fold chunk of the R = 1 kernel's operands as 16-column, 32-byte-row planes
    maps[4] = maps[0];
    maps[5] = maps[2];
    if (k_pad == 64) {
      s = encode_2d_sw64(&maps[4], ctx->tgt_hi.p, k_pad, n_pad, ks::kTcTileT, true, true);
      if (s != KS_OK) return s;
      maps[5] = ctx->tmB_f;
    } else if (k_pad == 32 && ctx->K <= 16) {
      s = encode_2d_sw64(&maps[4], ctx->tgt_lo.p, k_pad, n_pad, ks::kTcTileT, true, true);
      if (s != KS_OK) return s;
      maps[5] = ctx->tmB_f;
    }
  }
  if (ctx->r1) return eval_r1(ctx, maps, N, V);
  if (ctx->rv) return eval_rv(ctx, maps, N, V);

  ks::StreamK sk;
  sk.n_t = n_pad / ks::kTcTileT;
  sk.n_s = (int32_t)(ctx->m_pad / ks::fused_tc_tile_s(ctx->tc_vcc));
  sk.units = sk.n_t * (int64_t)sk.n_s;
  int64_t g = ctx->num_sms;
  if (g > sk.units) g = sk.units;
  sk.grid = (int32_t)g;
  KS_CUDA(ctx->partial.reserve((size_t)sk.grid * 2 * ks::kTcTileT * 32, st, false), "allocate partials");
  KS_CUDA(ctx->counters.reserve((size_t)sk.n_t, st, true), "allocate tile counters");

  ks::TcArgs a;
  a.N = N;
  a.k_pad = f16 ? k_pad / 2 : k_pad;  // in FP32 units: 64-byte chunks = k_pad / kTcKC
  a.R = ctx->R;
  a.f16 = f16 ? 1 : 0;
  a.tsc = ctx->tsc.p;
  a.wstat = ctx->tc_wstat ? ctx->wstat.p : nullptr;
  a.three = (ctx->prec_eff == KS_PREC_TF32) ? 0 : 1;
  a.aug = ctx->tc_aug;
  a.kcols = ctx->tc_kcols;
  a.kdims = ctx->tc_kdims;
  a.fold = ctx->tc_fold ? 1 : 0;
  a.amax = f16 ? ctx->amax.p : nullptr;
  a.c = ctx->c;
  a.K = ctx->K;
  a.wv = ctx->wv.p;
  a.wcol = ctx->wcol.p;
  a.vcc = ctx->tc_vcc;
  a.ares = ks::opt(KS_OPT_TARGET_RESIDENT, 1) ? 1 : 0;  // 0: reload the target operand per unit
  a.ar_stages = ks::opt(KS_OPT_AR_STAGES, 4) == 5 ? 5 : 4;
  {
    const int w = ks::opt(KS_OPT_WSLOTS, 0);
    a.wslots = (w >= 2 && w <= 4) ? w : 0;
  }
  a.dbg_skip_v = 0;
#if KS_DEBUG
  {
    const char* e = getenv("KS_TC_DEBUG_SKIP_V");
    // measurement builds only (wrong results): 1 no epilogue math, 4 W/na loaded once, 5 no S MMAs,
    // 6 one product, 7 no MMAs and no operand loads, 8 = 1 + 5, 9 = 1 + no operand loads, 10 = 1 + 7
    a.dbg_skip_v = e ? atoi(e) : 0;
    if (a.dbg_skip_v < 0 || a.dbg_skip_v > 10) a.dbg_skip_v = 0;
  }
#endif
  a.na = ctx->na.p;
  a.nb = ctx->nb.p;
  a.V = V;
  a.partial = ctx->partial.p;
  a.counters = ctx->counters.p;
  a.sk = sk;
  a.cta_times = nullptr;
  const char* dbg = ctx->cta_times_path.empty() ? nullptr : ctx->cta_times_path.c_str();
  const size_t n_dbg = (size_t)sk.grid * (2 + 20 * 5);  // CTA start/end + (KS_PROF builds) per-warp phase clocks
  if (dbg) {
    KS_CUDA(ctx->dbg_times.reserve(n_dbg, st, true), "allocate debug timers");
    a.cta_times = ctx->dbg_times.p;
  }
  for (int r_off = 0; r_off < ctx->r_pad;) {
    const int r_c = (ctx->r_pad - r_off >= 32) ? 32 : 16;
    a.r_c = r_c;
    a.r_off = r_off;
    a.r_valid = (ctx->R - r_off < r_c) ? (ctx->R - r_off) : r_c;
    if (f16) {  // FP16 V-MMA: one wcat map (hi and lo rows of the r_c columns in one box)
      s = encode_wcat(&maps[4], ctx->wt_hi.p, ctx->m_pad, ctx->r_pad, r_c, ks::kTcTileS);
      if (s != KS_OK) return s;
      maps[5] = maps[4];
    } else {
      s = encode_wt(&maps[4], ctx->wt_hi.p, ctx->m_pad, ctx->r_pad, r_c);
      if (s != KS_OK) return s;
      s = encode_wt(&maps[5], ctx->wt_lo.p, ctx->m_pad, ctx->r_pad, r_c);
      if (s != KS_OK) return s;
    }
    cudaEvent_t stop;
    s = timed_begin(ctx, &stop);
    if (s != KS_OK) return s;
    KS_CUDA(ks::launch_fused_tc(maps, a, st), "fused TC kernel launch");
    ctx->launches++;
    ctx->fused_launches++;
    ctx->last_grid = sk.grid;
    s = timed_end(ctx, stop);
    if (s != KS_OK) return s;
    r_off += r_c;
  }
  if (a.cta_times) {
    std::vector<unsigned long long> h(n_dbg);
    KS_CUDA(cudaMemcpyAsync(h.data(), a.cta_times, h.size() * 8, cudaMemcpyDeviceToHost, st), "copy debug timers");
    KS_CUDA(cudaStreamSynchronize(st), "synchronize");
    FILE* f = fopen(dbg, "a");
    if (f) {
      for (int i = 0; i < sk.grid; ++i) {
        fprintf(f, "%d %llu %llu", i, h[2 * i], h[2 * i + 1]);
        for (int k = 0; k < 20 * 5; ++k) fprintf(f, " %llu", h[2 * (size_t)sk.grid + (size_t)i * 100 + k]);
        fprintf(f, "\n");
      }
      fprintf(f, "--\n");
      fclose(f);
    }
  }
  return KS_OK;
}

// The TC path's per-eval target buffers for ctx->reserve_n targets at the current operand
// layout (ks_reserve; re-applied by ks_set_sources when the layout changes), so that no later
// ks_eval with N <= reserve_n allocates (CUDA-graph capture).
ks_status reserve_targets(ks_ctx* ctx) {
  if (ctx->reserve_n <= 0 || !ctx->have_src || ctx->path != KS_PATH_TC) return KS_OK;
  const int64_t n_pad = round_up(ctx->reserve_n, ks::kTcTileT);
  const size_t ntg = ctx->tc_f16 ? ((size_t)n_pad * ctx->k_pad + 1) / 2 : (size_t)n_pad * ctx->k_pad;
  cudaStream_t st = ctx->stream;
  KS_CUDA(ctx->tgt_hi.reserve(ntg, st, false), "allocate target hi");
  KS_CUDA(ctx->tgt_lo.reserve(ntg, st, false), "allocate target lo");
  KS_CUDA(ctx->nb.reserve((size_t)n_pad, st, false), "allocate target norms");
  KS_CUDA(ctx->tsc.reserve((size_t)n_pad, st, false), "allocate target scales");
  return KS_OK;
}

}  // namespace

extern "C" {

const char* ks_version(void) { return "ks-b200 0.1 (sm_100a)"; }

const char* ks_status_str(ks_status s) {
  switch (s) {
    case KS_OK: return "KS_OK";
    case KS_EINVAL: return "KS_EINVAL";
    case KS_ESTATE: return "KS_ESTATE";
    case KS_ENOMEM: return "KS_ENOMEM";
    case KS_ECUDA: return "KS_ECUDA";
    case KS_EUNSUPPORTED: return "KS_EUNSUPPORTED";
  }
  return "KS_UNKNOWN";
}

const char* ks_last_error(void) { return g_err.c_str(); }

ks_status ks_create(int K, float h, ks_ctx** out) {
  if (!out) return fail(KS_EINVAL, "out is NULL");
  *out = nullptr;
  if (K < 1 || K > 4096) return fail(KS_EINVAL, "K=%d outside [1, 4096]", K);
  if (!std::isfinite(h) || !(h > 0.f)) return fail(KS_EINVAL, "h=%g must be finite and > 0", (double)h);
  const double hd = (double)h;
  const double c = 1.4426950408889634 / (2.0 * hd * hd);
  if (!(c * 2.0 <= (double)FLT_MAX) || !(c >= (double)FLT_MIN))
    return fail(KS_EINVAL, "h=%g gives c=log2(e)/(2h^2)=%g outside FP32 range", (double)h, c);
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return cuda_fail(e, "cudaGetDevice (no CUDA device?)");
  cudaDeviceProp prop;
  e = cudaGetDeviceProperties(&prop, dev);
  if (e != cudaSuccess) return cuda_fail(e, "cudaGetDeviceProperties");
  if (!(prop.major == 10 && prop.minor == 0))
    return fail(KS_EUNSUPPORTED, "device %d is sm_%d%d; libks.so is built for sm_100a (B200) only", dev, prop.major,
                prop.minor);
  ks_ctx* ctx = new (std::nothrow) ks_ctx();
  if (!ctx) return fail(KS_ENOMEM, "host allocation of the context failed");
  ctx->device = dev;
  init_opts(ctx);
  ctx->num_sms = prop.multiProcessorCount;
  ctx->K = K;
  ctx->h = h;
  ctx->c = c;
  *out = ctx;
  g_err.clear();
  return KS_OK;
}

ks_status ks_destroy(ks_ctx* ctx) {
  if (!ctx) return KS_OK;
  set_device(ctx);
  cudaStreamSynchronize(ctx->stream);
  ctx->src.release();
  for (DBuf<float>* bptr : {&ctx->src_hi, &ctx->src_lo, &ctx->na, &ctx->wt_hi, &ctx->wt_lo, &ctx->wv, &ctx->tgt_hi,
                            &ctx->tgt_lo, &ctx->nb, &ctx->tsc})
    bptr->release();
  ctx->amax.release();
  ctx->wstat.release();
  ctx->mu.release();
  ctx->mean_part.release();
  ctx->mean_pmm.release();
  ctx->mean_pw.release();
  ctx->wcol.release();
  ctx->wcol_part.release();
  ctx->stats_counter.release();
  ctx->coop_bar.release();
  ctx->partial.release();
  ctx->counters.release();
  ctx->dbg_times.release();
  ctx->clk_buf.release();
  ctx->h_alpha.release();
  ctx->h_W.release();
  ctx->h_beta.release();
  ctx->h_V.release();
  for (cudaEvent_t ev : ctx->ev) cudaEventDestroy(ev);
  if (ctx->ev_copied) cudaEventDestroy(ctx->ev_copied);
  if (ctx->ev_stream) cudaEventDestroy(ctx->ev_stream);
  for (int c = 0; c < 4; ++c) {
    if (ctx->ev_bc[c]) cudaEventDestroy(ctx->ev_bc[c]);
    if (ctx->ev_v[c]) cudaEventDestroy(ctx->ev_v[c]);
  }
  if (ctx->copy_stream) {
    cudaStreamSynchronize(ctx->copy_stream);
    cudaStreamDestroy(ctx->copy_stream);
  }
  delete ctx;
  return KS_OK;
}

ks_status ks_set_precision(ks_ctx* ctx, ks_precision p) {
  if (check_ctx(ctx)) return KS_EINVAL;
  if (p != KS_PREC_AUTO && p != KS_PREC_FP32 && p != KS_PREC_3XTF32 && p != KS_PREC_TF32 && p != KS_PREC_3XF16)
    return fail(KS_EINVAL, "unknown precision %d", (int)p);
  ctx->prec_req = p;
  return KS_OK;
}

ks_status ks_set_option(ks_ctx* ctx, ks_option o, int value) {
  if (check_ctx(ctx)) return KS_EINVAL;
  const int i = (int)o;
  if (i < 1 || i >= KS_OPT_COUNT_) return fail(KS_EINVAL, "unknown option %d", i);
  if (value < kOpt[i].lo || value > kOpt[i].hi)
    return fail(KS_EINVAL, "option %d value %d outside [%d, %d]", i, value, kOpt[i].lo, kOpt[i].hi);
  ctx->opts.v[i] = value;
  return KS_OK;
}

ks_status ks_get_option(const ks_ctx* ctx, ks_option o, int* value) {
  if (check_ctx(ctx)) return KS_EINVAL;
  const int i = (int)o;
  if (!value) return fail(KS_EINVAL, "value is NULL");
  if (i < 1 || i >= KS_OPT_COUNT_) return fail(KS_EINVAL, "unknown option %d", i);
  *value = ctx->opts.v[i];
  return KS_OK;
}

ks_status ks_set_stream(ks_ctx* ctx, void* cuda_stream) {
  if (check_ctx(ctx)) return KS_EINVAL;
  cudaStream_t st = reinterpret_cast<cudaStream_t>(cuda_stream);
  if (st != ctx->stream) {
    // order the new stream after everything already enqueued on the old one (prepared sources,
    // buffers a later growth may free), so mixing streams across calls is safe
    ks_status s = set_device(ctx);
    if (s != KS_OK) return s;
    if (!ctx->ev_stream) KS_CUDA(cudaEventCreateWithFlags(&ctx->ev_stream, cudaEventDisableTiming), "create event");
    KS_CUDA(cudaEventRecord(ctx->ev_stream, ctx->stream), "cudaEventRecord");
    KS_CUDA(cudaStreamWaitEvent(st, ctx->ev_stream, 0), "cudaStreamWaitEvent");
    ctx->stream = st;
  }
  return KS_OK;
}

// NVTX range per ABI call (header-only NVTX 3: a no-op unless a profiler is attached), so an
// nsys / ncu capture shows ks_set_sources / ks_eval (and the host variants) around their launches
struct NvtxRange {
  explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
  ~NvtxRange() { nvtxRangePop(); }
};

ks_status ks_set_sources(ks_ctx* ctx, const float* alpha, const float* W, int64_t M, int R) {
  NvtxRange nvtx("ks_set_sources");
  if (check_ctx(ctx)) return KS_EINVAL;
  OptScope opt_scope(ctx);
  if (M < 0) return fail(KS_EINVAL, "M=%lld < 0", (long long)M);
  if (R < 1 || R > 256) return fail(KS_EINVAL, "R=%d outside [1, 256]", R);
  if (M > 0 && (!alpha || !W)) return fail(KS_EINVAL, "alpha/W is NULL with M=%lld", (long long)M);
  if (M > ((int64_t)1 << 31) - 256) return fail(KS_EINVAL, "M=%lld too large", (long long)M);
  int prec = ctx->prec_req;
  int path;
  if (prec == KS_PREC_AUTO) {
    // Measured on B200 (tools/msweep.py, SS7): the tcgen05 split-FP16 kernel is
    // faster for every source-set size once the target set is not tiny (M = 512, N = 65,536:
    // 0.044 vs 0.078 ms for set_sources + eval); the FP32 kernel only wins by ~8% when both
    // sets are ~1,000 points, and N is unknown here -- so AUTO is always the tensor-core path.
    path = KS_PATH_TC;
    prec = KS_PREC_3XF16;
  } else if (prec == KS_PREC_FP32) {
    if (ctx->K > 32 || R != 1)
      return fail(KS_EUNSUPPORTED, "FP32 path needs K <= 32 and R == 1 (K=%d, R=%d)", ctx->K, R);
    path = KS_PATH_FP32;
  } else {
    path = KS_PATH_TC;
  }
  ks_status s = set_device(ctx);
  if (s != KS_OK) return s;
  ctx->have_src = false;
  ctx->prec_eff = prec;
  s = (path == KS_PATH_TC) ? prepare_tc(ctx, alpha, W, M, R) : prepare_fp32(ctx, alpha, W, M);
  if (s != KS_OK) return s;
  ctx->path = path;
  ctx->prec_eff = prec;
  ctx->M = M;
  ctx->R = R;
  ctx->have_src = true;
  return reserve_targets(ctx);
}

ks_status ks_eval(ks_ctx* ctx, const float* beta, int64_t N, float* V) {
  NvtxRange nvtx("ks_eval");
  if (check_ctx(ctx)) return KS_EINVAL;
  OptScope opt_scope(ctx);
  if (N < 0) return fail(KS_EINVAL, "N=%lld < 0", (long long)N);
  if (!ctx->have_src) return fail(KS_ESTATE, "ks_eval before ks_set_sources");
  if (N == 0) return KS_OK;
  if (!beta || !V) return fail(KS_EINVAL, "beta/V is NULL with N=%lld", (long long)N);
  if (N > ((int64_t)1 << 31) - 256) return fail(KS_EINVAL, "N=%lld too large", (long long)N);
  ks_status s = set_device(ctx);
  if (s != KS_OK) return s;
  if (ctx->M == 0) {
    KS_CUDA(cudaMemsetAsync(V, 0, (size_t)N * ctx->R * sizeof(float), ctx->stream), "zero V");
    return KS_OK;
  }
  return (ctx->path == KS_PATH_TC) ? eval_tc(ctx, beta, N, V) : eval_fp32(ctx, beta, N, V);
}

ks_status ks_reserve(ks_ctx* ctx, int64_t N_max) {
  if (check_ctx(ctx)) return KS_EINVAL;
  OptScope opt_scope(ctx);
  if (N_max < 0) return fail(KS_EINVAL, "N_max < 0");
  ks_status s = set_device(ctx);
  if (s != KS_OK) return s;
  const int64_t n_t = (N_max + ks::kTcTileT - 1) / ks::kTcTileT;  // the finer of the two target tilings
  const int64_t g = (int64_t)ctx->num_sms;  // persistent grids are <= one CTA per SM
  const size_t per_cta = std::max((size_t)2 * ks::kTileT, (size_t)2 * ks::kTcTileT * 32);
  KS_CUDA(ctx->partial.reserve((size_t)g * per_cta, ctx->stream, false), "allocate partials");
  KS_CUDA(ctx->counters.reserve((size_t)(n_t > 0 ? n_t : 1), ctx->stream, true), "allocate tile counters");
  if (N_max > ctx->reserve_n) ctx->reserve_n = N_max;
  return reserve_targets(ctx);
}

namespace {
ks_status host_api_init(ks_ctx* ctx) {
  if (ctx->copy_stream) return KS_OK;
  KS_CUDA(cudaStreamCreateWithFlags(&ctx->copy_stream, cudaStreamNonBlocking), "create copy stream");
  KS_CUDA(cudaEventCreateWithFlags(&ctx->ev_copied, cudaEventDisableTiming), "create event");
  for (int c = 0; c < 4; ++c) {
    KS_CUDA(cudaEventCreateWithFlags(&ctx->ev_bc[c], cudaEventDisableTiming), "create event");
    KS_CUDA(cudaEventCreateWithFlags(&ctx->ev_v[c], cudaEventDisableTiming), "create event");
  }
  return KS_OK;
}
}  // namespace

ks_status ks_set_sources_host(ks_ctx* ctx, const float* alpha, const float* W, int64_t M, int R) {
  NvtxRange nvtx("ks_set_sources_host");
  if (check_ctx(ctx)) return KS_EINVAL;
  OptScope opt_scope(ctx);
  if (M < 0) return fail(KS_EINVAL, "M=%lld < 0", (long long)M);
  if (R < 1 || R > 256) return fail(KS_EINVAL, "R=%d outside [1, 256]", R);
  if (M > 0 && (!alpha || !W)) return fail(KS_EINVAL, "alpha/W is NULL with M=%lld", (long long)M);
  ks_status s = set_device(ctx);
  if (s != KS_OK) return s;
  const size_t na = (size_t)M * ctx->K, nw = (size_t)M * R;
  KS_CUDA(ctx->h_alpha.reserve(na ? na : 1, ctx->stream, false), "allocate alpha staging");
  KS_CUDA(ctx->h_W.reserve(nw ? nw : 1, ctx->stream, false), "allocate W staging");
  s = host_api_init(ctx);
  if (s != KS_OK) return s;
  if (M > 0) {
    KS_CUDA(cudaMemcpyAsync(ctx->h_alpha.p, alpha, na * 4, cudaMemcpyHostToDevice, ctx->stream), "copy alpha H2D");
    KS_CUDA(cudaMemcpyAsync(ctx->h_W.p, W, nw * 4, cudaMemcpyHostToDevice, ctx->stream), "copy W H2D");
  }
  KS_CUDA(cudaEventRecord(ctx->ev_copied, ctx->stream), "cudaEventRecord");
  s = ks_set_sources(ctx, ctx->h_alpha.p, ctx->h_W.p, M, R);
  if (s != KS_OK) return s;
  // return once the host buffers have been read; the source prep runs on (stream-ordered
  // before any later call on this context)
  KS_CUDA(cudaEventSynchronize(ctx->ev_copied), "synchronize");
  return KS_OK;
}

ks_status ks_eval_host(ks_ctx* ctx, const float* beta, int64_t N, float* V) {
  NvtxRange nvtx("ks_eval_host");
  if (check_ctx(ctx)) return KS_EINVAL;
  OptScope opt_scope(ctx);
  if (N < 0) return fail(KS_EINVAL, "N=%lld < 0", (long long)N);
  if (!ctx->have_src) return fail(KS_ESTATE, "ks_eval before ks_set_sources");
  if (N == 0) return KS_OK;
  if (!beta || !V) return fail(KS_EINVAL, "beta/V is NULL with N=%lld", (long long)N);
  ks_status s = set_device(ctx);
  if (s != KS_OK) return s;
  const size_t nb = (size_t)N * ctx->K, nv = (size_t)N * ctx->R;
  s = host_api_init(ctx);
  if (s != KS_OK) return s;
  KS_CUDA(ctx->h_beta.reserve(nb, ctx->stream, false), "allocate beta staging");
  KS_CUDA(ctx->h_V.reserve(nv, ctx->stream, false), "allocate V staging");
  // The uploads run on the copy stream (overlapping a source prep still in flight on `stream`;
  // the staging buffer's previous readers finished before the previous ks_eval_host returned).
  // Chunks: chunk c is evaluated while chunk c + 1 uploads and its V downloads while chunk c + 1
  // evaluates.  Default (KS_OPT_EVAL_CHUNK0 = 0) for N >= 2 waves of 128-target tiles: the
  // first chunk is exactly one wave (every CTA one whole target tile, no stream-K split) so the
  // first launch starts as soon as 148 tiles have arrived, and the rest is one launch (its upload
  // hides under the first one; measured at cfg3, SS7).  Smaller N, or
  // KS_OPT_EVAL_CHUNK0 = -1: up to 4 equal chunks of >= half a wave each.  KS_OPT_EVAL_CHUNK0 = t
  // > 0 makes the first chunk t tiles; KS_OPT_EVAL_CHUNKS = n forces n chunks in total.
  const int och = ctx->opts.v[KS_OPT_EVAL_CHUNKS], oc0 = ctx->opts.v[KS_OPT_EVAL_CHUNK0];
  const int64_t wave = (int64_t)ctx->num_sms * 128, half_wave = wave / 2;
  int64_t first = 0;  // targets in chunk 0 when it differs from the others
  if (oc0 > 0) first = (int64_t)oc0 * 128;
  else if (oc0 == 0 && N >= 2 * wave) first = wave;
  if (first >= N) first = 0;
  int nch;
  if (first > 0) nch = (och >= 2 && och <= 4) ? och : 2;
  else {
    nch = (int)(N / half_wave);
    if (och >= 1 && och <= 4) nch = och;
  }
  if (nch > 4) nch = 4;
  if (nch < 1) nch = 1;
  int64_t off[4] = {0, 0, 0, 0}, cnt[4] = {0, 0, 0, 0};
  {
    int64_t o = 0;
    int c0 = 0;
    if (first > 0) {
      cnt[0] = first;
      o = first;
      c0 = 1;
    }
    const int rest = nch - c0;
    const int64_t per = round_up((N - o + rest - 1) / rest, 128);
    for (int c = c0; c < nch; ++c) {
      off[c] = o;
      cnt[c] = (N - o < per) ? N - o : per;
      o += cnt[c];
    }
  }
  cudaEvent_t* evb = ctx->ev_bc;
  const int K = ctx->K, R = ctx->R;
  for (int c = 0; c < nch; ++c) {
    if (cnt[c] == 0) continue;
    KS_CUDA(cudaMemcpyAsync(ctx->h_beta.p + off[c] * K, beta + off[c] * K, (size_t)cnt[c] * K * 4,
                            cudaMemcpyHostToDevice, ctx->copy_stream),
            "copy beta H2D");
    KS_CUDA(cudaEventRecord(evb[c], ctx->copy_stream), "cudaEventRecord");
  }
  for (int c = 0; c < nch; ++c) {
    if (cnt[c] == 0) continue;
    KS_CUDA(cudaStreamWaitEvent(ctx->stream, evb[c], 0), "cudaStreamWaitEvent");
    s = ks_eval(ctx, ctx->h_beta.p + off[c] * K, cnt[c], ctx->h_V.p + off[c] * R);
    if (s != KS_OK) return s;
    KS_CUDA(cudaEventRecord(ctx->ev_v[c], ctx->stream), "cudaEventRecord");
    KS_CUDA(cudaStreamWaitEvent(ctx->copy_stream, ctx->ev_v[c], 0), "cudaStreamWaitEvent");
    KS_CUDA(cudaMemcpyAsync(V + off[c] * R, ctx->h_V.p + off[c] * R, (size_t)cnt[c] * R * 4,
                            cudaMemcpyDeviceToHost, ctx->copy_stream),
            "copy V D2H");
  }
  KS_CUDA(cudaStreamSynchronize(ctx->copy_stream), "synchronize");
  KS_CUDA(cudaStreamSynchronize(ctx->stream), "synchronize");
  return KS_OK;
}

ks_status ks_get_info(const ks_ctx* ctx, ks_info* out) {
  if (!ctx || !out) return fail(KS_EINVAL, "ctx/out is NULL");
  memset(out, 0, sizeof *out);
  out->path = ctx->have_src ? ctx->path : KS_PATH_NONE;
  out->precision = ctx->have_src ? ctx->prec_eff : ctx->prec_req;
  out->k_pad = ctx->k_pad;
  const bool tc = ctx->have_src && ctx->path == KS_PATH_TC;
  out->tile_t = tc ? ks::kTcTileT : ks::kTileT;
  out->tile_s = tc ? (ctx->r1 ? 128 : ctx->rv ? ks::kRvTileS : ks::fused_tc_tile_s(ctx->tc_vcc)) : ks::kTileS;
  out->num_ctas = ctx->last_grid;
  out->stages = !ctx->k_pad ? 0
                : tc && ctx->r1 ? ks::fused_r1_stages(ctx->K, ctx->opts.v[KS_OPT_NARROW_PLANES] != 0)
                : (tc ? ks::fused_tc_stages(ctx->tc_vcc, ctx->tc_f16 != 0, ctx->tc_f16 ? ctx->k_pad / 2 : ctx->k_pad,
                                            ctx->r_pad >= 32 ? 32 : 16)
                      : ks::fused_fp32_stages(ctx->k_pad));
  out->num_sms = ctx->num_sms;
  out->m = ctx->M;
  out->m_pad = ctx->m_pad;
  out->r = ctx->R;
  out->launches = ctx->launches;
  out->fused_launches = ctx->fused_launches;
  out->c_log2 = ctx->c;
  out->kernel = !ctx->have_src ? 0 : ctx->path == KS_PATH_FP32 ? 1 : ctx->r1 ? 3 : ctx->rv ? 4 : 2;
  out->exp_poly = ctx->r1   ? ks::r1_poly_for(ctx->opts.v[KS_OPT_EXP_POLY])
                  : ctx->rv ? ks::rv_poly_for(ctx->opts.v[KS_OPT_EXP_POLY])
                            : ctx->opts.v[KS_OPT_EXP_POLY];
  out->r1_epilogue = ctx->r1 ? ctx->opts.v[KS_OPT_R1_EPILOGUE] : -1;
  return KS_OK;
}

ks_status ks_clock_read(ks_ctx* ctx, double* sm_ghz, int* ctas) {
  if (check_ctx(ctx)) return KS_EINVAL;
  if (!sm_ghz || !ctas) return fail(KS_EINVAL, "sm_ghz/ctas is NULL");
  if (ctx->clk_ctas <= 0 || !ctx->clk_buf.p) return fail(KS_ESTATE, "no measured launch (KS_OPT_MEASURE_CLOCK)");
  ks_status s = set_device(ctx);
  if (s != KS_OK) return s;
  std::vector<unsigned long long> h((size_t)ctx->clk_ctas * 4);
  KS_CUDA(cudaMemcpyAsync(h.data(), ctx->clk_buf.p, h.size() * 8, cudaMemcpyDeviceToHost, ctx->stream),
          "copy clock records");
  KS_CUDA(cudaStreamSynchronize(ctx->stream), "synchronize");
  double acc = 0.0;
  int n = 0;
  for (int b = 0; b < ctx->clk_ctas; ++b) {
    const double dt = (double)(h[4 * b + 2] - h[4 * b]), dc = (double)(h[4 * b + 3] - h[4 * b + 1]);
    if (dt > 0.0) {
      acc += dc / dt;
      ++n;
    }
  }
  if (n == 0) return fail(KS_ESTATE, "empty clock records");
  *sm_ghz = acc / n;
  *ctas = n;
  return KS_OK;
}

ks_status ks_timing_enable(ks_ctx* ctx, int on) {
  if (check_ctx(ctx)) return KS_EINVAL;
  ctx->timing = on != 0;
  return KS_OK;
}

ks_status ks_timing_read(ks_ctx* ctx, double* total_ms, int64_t* launches, int reset) {
  if (check_ctx(ctx)) return KS_EINVAL;
  if (!total_ms || !launches) return fail(KS_EINVAL, "total_ms/launches is NULL");
  ks_status s = set_device(ctx);
  if (s != KS_OK) return s;
  KS_CUDA(cudaStreamSynchronize(ctx->stream), "synchronize");
  double tot = 0.0;
  for (size_t i = 0; i < ctx->ev_used; ++i) {
    float ms = 0.f;
    KS_CUDA(cudaEventElapsedTime(&ms, ctx->ev[2 * i], ctx->ev[2 * i + 1]), "cudaEventElapsedTime");
    tot += ms;
  }
  *total_ms = tot;
  *launches = (int64_t)ctx->ev_used;
  if (reset) ctx->ev_used = 0;
  return KS_OK;
}

}  // extern "C"
