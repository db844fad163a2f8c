// ks_prep.cu -- source preparation (scope row a1).
//
// Paper: Alg.1 l.3 computes vec_alpha = [||alpha_0||^2 ... ||alpha_{M-1}||^2]
// for the norm identity Eq.3.  The paper does
// not say where or how.  Here it runs once per ks_set_sources, on the device:
//   1. mu = mean of the sources (FP64 accumulation, fixed order) -- centring
//      is exact for the Gaussian (it depends on alpha - beta only) and shrinks
//      the cancellation of Eq.3 in FP32 (SS3, reading Q8/Q11);
//   2. per source: alpha_hat = alpha - mu (FP32), n = ||alpha_hat||^2 (FP64
//      accumulate), stored prescaled for the ex2-based exponent:
//      a = RN(2c * alpha_hat), na = RN(-c * n), c = log2(e)/(2h^2);
//      layout dimension-major so one TMA box brings a source tile's
//      coordinates, norms and weights into shared memory.
#include "ks_internal.h"

#include <cstdlib>

namespace ks {

// Source statistics in one launch.  Each block reduces a contiguous chunk of
// rows in a fixed order: FP64 column sums, FP32 column min/max and (R = 1 log-
// weight mode) max |W_i| and "any W_i < 0 or NaN".  The last block to finish
// (arrival counter, reset for the next call) reduces the block partials in
// fixed block order -- the result is bitwise independent of which block is
// last -- and writes
//   mu[d]   = sum_i alpha_id / M (FP32; 0 for padding dims),
//   amax    = max_{i,d} |fl(alpha_id - mu_d)| as FP32 bits, from the column
//             extremes: fl(x - mu) is monotone in x and RN is sign-symmetric, so
//             max(fl(max_d - mu_d), fl(mu_d - min_d)) is that maximum exactly,
//   wstat   = {bits of max |W_i|, any W_i < 0 or NaN}.
// For K <= 256 the 256 threads form rpp = 256/K row lanes x K dims (coalesced
// reads); the rpp lane partials of a dim are combined in lane order.  For
// K > 256 thread t owns dims t, t+256, ...  The final reduction uses the same
// thread layout over the block partials.
__global__ void source_stats_kernel(const float* __restrict__ alpha, const float* __restrict__ W, int64_t M, int K,
                                    int k_pad, int nparts, double* __restrict__ part, float* __restrict__ pmm,
                                    unsigned* __restrict__ pw, unsigned* __restrict__ counter,
                                    float* __restrict__ mu, unsigned* __restrict__ amax,
                                    unsigned* __restrict__ wstat) {
  __shared__ double red[256];
  __shared__ float rmn[256], rmx[256];
  __shared__ unsigned s_w[2], s_amax;
  __shared__ bool s_last;
  pdl_trigger();  // the source prep may start its CTAs (it waits for this grid to complete)
  const int b = blockIdx.x;
  const int t = threadIdx.x;
  const int64_t chunk = (M + nparts - 1) / nparts;
  const int64_t r0 = b * chunk < M ? b * chunk : M;
  const int64_t r1 = (r0 + chunk < M) ? r0 + chunk : M;
  if (t == 0) {
    s_w[0] = 0u;
    s_w[1] = 0u;
    s_amax = 0u;
  }
  if (K <= 256) {
    const int rpp = 256 / K;
    const int ro = t / K, d = t % K;
    double s = 0.0;
    float mn = INFINITY, mx = -INFINITY;
    if (ro < rpp)
#pragma unroll 8
      for (int64_t r = r0 + ro; r < r1; r += rpp) {
        const float x = alpha[r * K + d];
        s += (double)x;
        mn = fminf(mn, x);
        mx = fmaxf(mx, x);
      }
    red[t] = s;
    rmn[t] = mn;
    rmx[t] = mx;
    __syncthreads();
    if (t < K) {
      double acc = 0.0;
      for (int q = 0; q < rpp; ++q) {
        acc += red[q * K + t];
        mn = fminf(mn, rmn[q * K + t]);
        mx = fmaxf(mx, rmx[q * K + t]);
      }
      part[(int64_t)b * K + t] = acc;
      pmm[((int64_t)b * K + t) * 2] = mn;
      pmm[((int64_t)b * K + t) * 2 + 1] = mx;
    }
  } else {
    for (int d = t; d < K; d += blockDim.x) {
      double s = 0.0;
      float mn = INFINITY, mx = -INFINITY;
#pragma unroll 8
      for (int64_t r = r0; r < r1; ++r) {
        const float x = alpha[r * K + d];
        s += (double)x;
        mn = fminf(mn, x);
        mx = fmaxf(mx, x);
      }
      part[(int64_t)b * K + d] = s;
      pmm[((int64_t)b * K + d) * 2] = mn;
      pmm[((int64_t)b * K + d) * 2 + 1] = mx;
    }
  }
  if (wstat != nullptr) {  // R = 1 weight statistics of the same rows
    float m = 0.f;
    unsigned neg = 0u;
#pragma unroll 4
    for (int64_t r = r0 + t; r < r1; r += blockDim.x) {
      const float w = W[r];
      m = fmaxf(m, fabsf(w));
      neg |= (w < 0.f || w != w) ? 1u : 0u;  // NaN weights take the general path
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, o));
      neg |= __shfl_xor_sync(0xffffffffu, neg, o);
    }
    __syncthreads();  // s_w initialised
    if ((t & 31) == 0) {
      atomicMax(&s_w[0], __float_as_uint(m));
      atomicOr(&s_w[1], neg);
    }
  }
  __syncthreads();
  if (wstat != nullptr && t == 0) {
    pw[2 * b] = s_w[0];
    pw[2 * b + 1] = s_w[1];
  }
  if (counter == nullptr) {  // K > 32: stats_final_kernel reduces the partials (one block per dim)
    if (b == 0 && t == 0 && amax != nullptr) *amax = 0u;
    return;
  }
  // publish the partials, then elect the last block
  __threadfence();
  __syncthreads();
  if (t == 0) s_last = atomicAdd(counter, 1u) == (unsigned)(nparts - 1);
  __syncthreads();
  if (!s_last) return;
  __threadfence();
  // fixed-order reduction of the block partials, all threads busy: for K <= 256,
  // rpp threads per dim stride over the blocks (loads unrolled), then thread d
  // combines its dim's rpp partials in order; for K > 256 a thread per dim
  for (int d0 = 0; d0 < K; d0 += 256) {
    const int kk = K - d0 < 256 ? K - d0 : 256;  // dims in this pass
    const int rpp = 256 / kk;
    const int ro = t / kk, d = d0 + t % kk;
    double s = 0.0;
    float mn = INFINITY, mx = -INFINITY;
    if (ro < rpp)
#pragma unroll 8
      for (int q = ro; q < nparts; q += rpp) {
        s += __ldcg(&part[(int64_t)q * K + d]);
        const float2 m2 = __ldcg(reinterpret_cast<const float2*>(&pmm[((int64_t)q * K + d) * 2]));
        mn = fminf(mn, m2.x);
        mx = fmaxf(mx, m2.y);
      }
    __syncthreads();  // red/rmn/rmx free
    red[t] = s;
    rmn[t] = mn;
    rmx[t] = mx;
    __syncthreads();
    if (t < kk) {
      double acc = 0.0;
      for (int q = 0; q < rpp; ++q) {
        acc += red[q * kk + t];
        mn = fminf(mn, rmn[q * kk + t]);
        mx = fmaxf(mx, rmx[q * kk + t]);
      }
      const float m = M > 0 ? (float)(acc / (double)M) : 0.f;
      mu[d0 + t] = m;
      if (M > 0) {
        // NaN coordinates give a NaN mean; fmaxf(NaN, 0) = 0 then ignores them
        const float a = fmaxf(fmaxf(mx - m, m - mn), 0.f);
        atomicMax(&s_amax, __float_as_uint(a));
      }
    }
  }
  for (int d = K + t; d < k_pad; d += blockDim.x) mu[d] = 0.f;
  if (wstat != nullptr && t < 32) {
    unsigned m = 0u, neg = 0u;
    for (int q = t; q < nparts; q += 32) {
      m = max(m, __ldcg(&pw[2 * q]));
      neg |= __ldcg(&pw[2 * q + 1]);
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      m = max(m, __shfl_xor_sync(0xffffffffu, m, o));
      neg |= __shfl_xor_sync(0xffffffffu, neg, o);
    }
    if (t == 0) {
      wstat[0] = m;  // non-negative FP32 values order as their bit patterns
      wstat[1] = neg;
    }
  }
  __syncthreads();
  if (t == 0) {
    if (amax != nullptr) *amax = s_amax;
    *counter = 0u;  // ready for the next call (stream order)
  }
}

bool pdl_enabled() {
  static const bool on = [] {
    const char* e = getenv("KS_PDL");
    return !(e && e[0] == '0');
  }();
  return on;
}

// K > 32: the block partials are reduced by K + 1 blocks instead of the last one -- block d
// sums dimension d over all partials (thread t: partials t, t + 256, ... in order, then a
// fixed shared-memory tree), writes mu[d] and folds its max |fl(alpha_d - mu_d)| into amax
// (atomicMax: order-independent; zeroed by the partial kernel); block K writes the padding
// dims of mu and the weight statistics.
__global__ void __launch_bounds__(256) stats_final_kernel(int64_t M, int K, int k_pad, int nparts,
                                                          const double* __restrict__ part,
                                                          const float* __restrict__ pmm,
                                                          const unsigned* __restrict__ pw, float* __restrict__ mu,
                                                          unsigned* __restrict__ amax, unsigned* __restrict__ wstat) {
  __shared__ double red[256];
  __shared__ float rmn[256], rmx[256];
  const int d = blockIdx.x, t = threadIdx.x;
  if (d == K) {
    for (int e = K + t; e < k_pad; e += blockDim.x) mu[e] = 0.f;
    if (wstat != nullptr && t < 32) {
      unsigned m = 0u, neg = 0u;
      for (int q = t; q < nparts; q += 32) {
        m = max(m, pw[2 * q]);
        neg |= pw[2 * q + 1];
      }
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) {
        m = max(m, __shfl_xor_sync(0xffffffffu, m, o));
        neg |= __shfl_xor_sync(0xffffffffu, neg, o);
      }
      if (t == 0) {
        wstat[0] = m;
        wstat[1] = neg;
      }
    }
    return;
  }
  double s = 0.0;
  float mn = INFINITY, mx = -INFINITY;
#pragma unroll 4
  for (int q = t; q < nparts; q += blockDim.x) {
    s += part[(int64_t)q * K + d];
    const float2 m2 = *reinterpret_cast<const float2*>(&pmm[((int64_t)q * K + d) * 2]);
    mn = fminf(mn, m2.x);
    mx = fmaxf(mx, m2.y);
  }
  red[t] = s;
  rmn[t] = mn;
  rmx[t] = mx;
  __syncthreads();
  for (int o = 128; o > 0; o >>= 1) {
    if (t < o) {
      red[t] += red[t + o];
      rmn[t] = fminf(rmn[t], rmn[t + o]);
      rmx[t] = fmaxf(rmx[t], rmx[t + o]);
    }
    __syncthreads();
  }
  if (t == 0) {
    const float m = M > 0 ? (float)(red[0] / (double)M) : 0.f;
    mu[d] = m;
    // NaN coordinates give a NaN mean; fmaxf(NaN, 0) = 0 then ignores them
    if (M > 0 && amax != nullptr) atomicMax(amax, __float_as_uint(fmaxf(fmaxf(rmx[0] - m, m - rmn[0]), 0.f)));
  }
}

cudaError_t launch_source_stats(const float* alpha, const float* W, int64_t M, int K, int k_pad, int nparts,
                                double* part, float* pmm, unsigned* pw, unsigned* counter, float* mu,
                                unsigned* amax, unsigned* wstat, cudaStream_t st) {
  const bool split = K > 32 || nparts > 256;  // reduce the partials with K + 1 blocks (a parallel tree per dim)
  source_stats_kernel<<<nparts, 256, 0, st>>>(alpha, W, M, K, k_pad, nparts, part, pmm, pw, split ? nullptr : counter,
                                              mu, amax, wstat);
  if (split) stats_final_kernel<<<K + 1, 256, 0, st>>>(M, K, k_pad, nparts, part, pmm, pw, mu, amax, wstat);
  return cudaGetLastError();
}

// One thread per (padded) source column.
__global__ void prep_fp32_kernel(const float* __restrict__ alpha, const float* __restrict__ W, int64_t M,
                                 int64_t m_pad, int K, int k_pad, const float* __restrict__ mu, double c,
                                 float* __restrict__ src) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= m_pad) return;
  const bool live = i < M;
  const double c2 = 2.0 * c;
  double n = 0.0;
  for (int d = 0; d < k_pad; ++d) {
    float x = 0.f;
    if (live && d < K) x = alpha[i * K + d] - mu[d];  // FP32 centring, same op as the target side
    n += (double)x * (double)x;
    src[(int64_t)d * m_pad + i] = (float)(c2 * (double)x);
  }
  src[(int64_t)k_pad * m_pad + i] = live ? (float)(-c * n) : 0.f;
  src[(int64_t)(k_pad + 1) * m_pad + i] = live ? W[i] : 0.f;
}

cudaError_t launch_prep_fp32(const float* alpha, const float* W, int64_t M, int64_t m_pad, int K, int k_pad,
                             const float* mu, double c, float* src, cudaStream_t st) {
  if (m_pad == 0) return cudaSuccess;
  const int bs = 256;
  const int64_t nb = (m_pad + bs - 1) / bs;
  prep_fp32_kernel<<<(unsigned)nb, bs, 0, st>>>(alpha, W, M, m_pad, K, k_pad, mu, c, src);
  return cudaGetLastError();
}

}  // namespace ks
