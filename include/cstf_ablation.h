/* include/cstf_ablation.h -- BENCH-ONLY C ABI: the ADMM variants of the paper's
 * Fig. 4 ablation (Sec. 5.2; Fig. 4), built as
 * libcstf_ablation.so next to libcstf.so.  Nothing in libcstf calls these; they
 * exist so bench.py --ablation and tests/test_gpu_ablation.py can time and check
 * the paper's baseline against its two optimisations on B200.
 *
 * Every arm runs `max_iter` passes of generic ADMM (Alg. 2) with
 * tol = 0 (the paper's timing protocol, L930-933) on row-major FP64 I x R
 * device matrices, in place on d_H / d_U, stream-ordered on `stream`:
 *   rho = tr(S)/R;  L = chol(S + rho I)
 *   repeat: H0 <- H;  T <- M + rho (H + U);  H~ <- T (L L^T)^{-1};
 *           H <- max(0, H~ - U);  U <- U + H - H~;
 *           r = ||H - H~||^2, s = ||H - H0||^2, nH = ||H||^2, nU = ||U||^2
 * The arms differ only in HOW (the arithmetic is the same up to rounding order):
 *   CSTF_ABL_BASELINE  one kernel / library call per element-wise operation of
 *                      Alg. 2 (H0 copy, two DGEAM, prox, dual, residual sums)
 *                      and two cuBLAS DTRSM per pass (per-iteration triangular
 *                      solves, L566 / L576)
 *   CSTF_ABL_OF        operation fusion only (Sec. 4.3.1): one fused
 *                      kernel forms T, one fused kernel does prox + dual +
 *                      residual partial sums; still two DTRSM per pass
 *   CSTF_ABL_PI        pre-inversion only (Sec. 4.3.2): Inv = (L L^T)^-1
 *                      once, one cuBLAS DGEMM per pass; element-wise steps
 *                      unfused as in the baseline
 *   CSTF_ABL_OF_PI     both: fused T kernel, DGEMM with Inv, fused epilogue
 *                      kernel (the paper's cuADMM shape, Alg. 3)
 * (libcstf's own one-launch-per-pass and row-resident kernels are the further
 * arms; bench.py calls them through cstf_admm_update.)
 *   stats_out  host double[6]: iters, rho, r, s, nH, nU of the last pass (may be NULL)
 * Returns 0 on success, nonzero on a CUDA / cuBLAS error or R outside [1, 64]
 * (message via cstf_ablation_last_error).  BLOCKING at the end (reads the stats). */
#ifndef CSTF_ABLATION_H
#define CSTF_ABLATION_H
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

typedef enum { CSTF_ABL_BASELINE = 0, CSTF_ABL_OF = 1, CSTF_ABL_PI = 2, CSTF_ABL_OF_PI = 3 } cstf_ablation_arm;

int cstf_ablation_admm(int arm, const double* d_M, const double* d_S, double* d_H, double* d_U, int64_t I, int R,
                       int max_iter, double* stats_out, void* stream);
const char* cstf_ablation_last_error(void);
/* kernel launches + cuBLAS calls issued by the last cstf_ablation_admm call */
int64_t cstf_ablation_last_calls(void);
/* Measured FP64 tensor-path peak of the current device in TFLOP/s: best of 3
 * launches of a chain-only mma.sync.m8n8k4.f64 kernel (SASS DMMA.8x8x4; 8
 * independent accumulators per warp, 8 CTAs of 256 threads per SM, ~10 ms each)
 * on `stream`, after a warm-up launch.  The roofline denominator of the ADMM
 * (SURVEY s8(d)).  Blocking; allocates and frees a small buffer.  Returns a
 * negative value on any CUDA error. */
double cstf_ablation_fp64_peak(void* stream);

#ifdef __cplusplus
}
#endif
#endif
