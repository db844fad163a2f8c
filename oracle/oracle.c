/*
 * oracle.c -- CPU reference ("oracle") for Gaussian kernel summation.
 *
 * TEST INFRASTRUCTURE ONLY.  Nothing on the product path (libks.so, the
 * Python binding, the CUDA kernels) may include, link, load or call this
 * file.  Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs use it.  It shares no code, header, constant or
 * helper with csrc/.
 *
 * What it computes is the plain definition of the method, nothing more:
 *
 *   Eq.1 (SS I):
 *       K(alpha_i, beta_j) = exp( -||alpha_i - beta_j||_2^2 / (2 h^2) )
 *   Eq.2 (SS I):
 *       V_j = sum_i K(alpha_i, beta_j) * W_i
 *
 * with the readings listed in DESIGN.md SS3 (Q1: the bandwidth is 2h^2;
 * Q2: W weights the sources alpha, V is indexed by the targets beta;
 * Q3: M sources and N targets may differ; Q14: i = j self terms are
 * included; Q15: no normalisation; Q17: R weight columns are independent,
 * V[:, r] = sum_i K(alpha_i, beta_j) W[i, r]).
 *
 * Deliberately NOT the paper's fast formulation: the squared distance is
 * formed from direct coordinate differences (never the norm identity Eq.3),
 * the exponential is libm exp() in double, and the sum over sources runs in
 * ascending i.  Everything is FP64; the FP32 inputs are widened exactly.
 *
 * Parallelism: OpenMP over targets only.  Each target's arithmetic is a
 * fixed sequential loop, so the result is bitwise identical for any thread
 * count.
 *
 * Pins (what makes this trustworthy without another implementation) are in
 * tests/test_oracle_pins.py; SS4.
 */
#include <math.h>
#include <stdint.h>
#include <stddef.h>

#ifdef _OPENMP
#include <omp.h>
#endif

/* Return codes: 0 ok, 1 invalid argument. */
int oracle_eval(const float *alpha,   /* [M][K] row-major sources        */
                const float *W,       /* [M][R] row-major weights        */
                int64_t M, int R,
                const float *beta,    /* [N][K] row-major targets        */
                int64_t N, int K,
                double h,             /* bandwidth (Eq.1)                */
                const int64_t *J,     /* target subset, or NULL = 0..N-1 */
                int64_t nJ,           /* |J| (ignored if J == NULL)      */
                double *V,            /* out [nJ][R]                     */
                double *S)            /* out [nJ][R] sum_i K|W|, or NULL */
{
    if (M < 0 || N < 0 || K < 1 || R < 1) return 1;
    if (!(h > 0.0)) return 1;
    const int64_t nt = J ? nJ : N;
    if (nt < 0) return 1;
    const double den = 2.0 * h * h;          /* Eq.1 denominator 2h^2 */

    int64_t t;
#pragma omp parallel for schedule(static)
    for (t = 0; t < nt; ++t) {
        const int64_t j = J ? J[t] : t;
        double *v = V + t * (int64_t)R;
        double *s = S ? S + t * (int64_t)R : NULL;
        for (int r = 0; r < R; ++r) { v[r] = 0.0; if (s) s[r] = 0.0; }
        if (j < 0 || j >= N) continue;       /* out-of-range index: zeros */
        const float *b = beta + j * (int64_t)K;
        for (int64_t i = 0; i < M; ++i) {    /* Eq.2: ascending sum over sources */
            const float *a = alpha + i * (int64_t)K;
            double d2 = 0.0;                 /* ||alpha_i - beta_j||^2, direct */
            for (int d = 0; d < K; ++d) {
                const double diff = (double)b[d] - (double)a[d];
                d2 += diff * diff;
            }
            const double k = exp(-d2 / den); /* Eq.1 */
            const float *w = W + i * (int64_t)R;
            for (int r = 0; r < R; ++r) {
                v[r] += k * (double)w[r];
                if (s) s[r] += k * fabs((double)w[r]);
            }
        }
    }
    return 0;
}

/* Threads OpenMP will use for oracle_eval (reported as cpu_baseline.cores). */
int oracle_num_threads(void)
{
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}

void oracle_set_num_threads(int n)
{
#ifdef _OPENMP
    if (n > 0) omp_set_num_threads(n);
#else
    (void)n;
#endif
}
