// BENCH-ONLY: the ADMM arms of the paper's Fig. 4 ablation (include/cstf_ablation.h).
// PAPER.md Sec. 5.2 (L933-958): a generic cuBLAS ADMM (Alg. 2: separate
// element-wise calls, per-iteration triangular solves) against operation fusion
// (Sec. 4.3.1), pre-inversion (Sec. 4.3.2) and both (Alg. 3,
// L630-660).  These are plain FP64 CUDA kernels + cuBLAS DGEAM / DTRSM / DGEMM, i.e.
// the library-call shape the paper measured, run on B200; libcstf's own kernels are
// the further arms.  Not linked into libcstf.
#include <cublas_v2.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include <algorithm>
#include <string>

#include "../../include/cstf_ablation.h"

namespace {

thread_local std::string g_err;
thread_local int64_t g_calls = 0;

int err(const std::string& m) {
  g_err = m;
  return 1;
}
#define ACU(x)                                                                         \
  do {                                                                                 \
    cudaError_t e_ = (x);                                                              \
    if (e_ != cudaSuccess) return err(std::string(#x) + ": " + cudaGetErrorString(e_)); \
  } while (0)
#define ABL(x)                                                                   \
  do {                                                                           \
    cublasStatus_t s_ = (x);                                                     \
    if (s_ != CUBLAS_STATUS_SUCCESS) return err(std::string(#x) + ": cublas " + std::to_string((int)s_)); \
    g_calls++;                                                                   \
  } while (0)
#define LAUNCHED()                        \
  do {                                    \
    g_calls++;                            \
    ACU(cudaGetLastError());              \
  } while (0)

constexpr int kT = 256;

// One CTA (R <= 64): rho = tr(S)/R, L = chol(S + rho I) (column-major, for cuBLAS),
// optionally Inv = L^-T L^-1.  consts = {1, rho, 0, -1}.  flag = 1 if not SPD.
__global__ void k_chol(const double* __restrict__ S, int R, int want_inv, double* __restrict__ Lc,
                       double* __restrict__ Inv, double* __restrict__ consts, int* __restrict__ flag) {
  extern __shared__ double sm_chol[];
  double* A = sm_chol;                         // [R][R]
  double* X = sm_chol + R * R;                 // [R][R]
  __shared__ double rho;
  const int t = threadIdx.x;
  if (t == 0) {
    double tr = 0.0;
    for (int i = 0; i < R; i++) tr += S[i * R + i];
    rho = tr / R;
  }
  __syncthreads();
  for (int x = t; x < R * R; x += blockDim.x) A[x] = S[x] + ((x / R == x % R) ? rho : 0.0);
  __syncthreads();
  for (int k = 0; k < R; k++) {               // right-looking, lower triangle in A
    if (t == 0) A[k * R + k] = A[k * R + k] > 0.0 ? sqrt(A[k * R + k]) : -1.0;
    __syncthreads();
    const double d = A[k * R + k];
    for (int i = k + 1 + t; i < R; i += blockDim.x) A[i * R + k] = A[i * R + k] / d;
    __syncthreads();
    for (int x = t; x < (R - k - 1) * (R - k - 1); x += blockDim.x) {
      const int i = k + 1 + x / (R - k - 1), j = k + 1 + x % (R - k - 1);
      if (j <= i) A[i * R + j] -= A[i * R + k] * A[j * R + k];
    }
    __syncthreads();
  }
  bool bad = !(rho > 0.0);
  for (int k = 0; k < R; k++) bad = bad || !(A[k * R + k] > 0.0);
  if (t == 0) {
    *flag = bad ? 1 : 0;
    consts[0] = 1.0; consts[1] = rho; consts[2] = 0.0; consts[3] = -1.0;
  }
  for (int x = t; x < R * R; x += blockDim.x) {
    const int i = x / R, j = x % R;
    Lc[i + j * R] = (j <= i) ? A[i * R + j] : 0.0;      // column-major L
  }
  if (!want_inv) return;
  for (int j = t; j < R; j += blockDim.x) {    // column j of L^-1 (forward substitution)
    for (int i = 0; i < R; i++) X[i * R + j] = 0.0;
    X[j * R + j] = 1.0 / A[j * R + j];
    for (int i = j + 1; i < R; i++) {
      double s = 0.0;
      for (int k = j; k < i; k++) s += A[i * R + k] * X[k * R + j];
      X[i * R + j] = -s / A[i * R + i];
    }
  }
  __syncthreads();
  for (int x = t; x < R * R; x += blockDim.x) {  // Inv = L^-T L^-1 (symmetric)
    const int a = x / R, b = x % R;
    double s = 0.0;
    for (int k = a > b ? a : b; k < R; k++) s += X[k * R + a] * X[k * R + b];
    Inv[x] = s;
  }
}

// Element-wise kernels: 16-byte (double2) accesses over the flat I x R array, grid
// = 16 CTAs per SM; every thread loads kU pairs (one grid stride apart) before it
// computes and stores any of them, so enough loads are in flight to stream at the
// HBM rate (one pair per iteration left the fused epilogue at 1.6 TB/s: ncu
// long-scoreboard 197 cycles per issue).  An odd element count leaves one scalar
// tail element for thread 0 of CTA 0.
constexpr int kU = 4;
__device__ __forceinline__ double2 ld2(const double* p, int64_t x) { return reinterpret_cast<const double2*>(p)[x]; }
__device__ __forceinline__ void st2(double* p, int64_t x, double a, double b) {
  reinterpret_cast<double2*>(p)[x] = make_double2(a, b);
}
__device__ __forceinline__ double prox0(double v) { return v > 0.0 ? v : 0.0; }
#define ABL_LOOP_BEGIN                                                               \
  const int64_t n2 = n >> 1, stride = (int64_t)gridDim.x * kT;                       \
  for (int64_t x0 = blockIdx.x * (int64_t)kT + threadIdx.x; x0 < n2; x0 += kU * stride) {
#define ABL_LOOP_END }
#define ABL_FOR_K _Pragma("unroll") for (int k = 0; k < kU; k++)
#define ABL_X const int64_t x = x0 + k * stride; if (x < n2)
#define ABL_TAIL if ((n & 1) && blockIdx.x == 0 && threadIdx.x == 0)

// ---- unfused element-wise steps of Alg. 2 (one call per operation)
__global__ void k_prox(const double* __restrict__ Ht, const double* __restrict__ U, double* __restrict__ H, int64_t n) {
  ABL_LOOP_BEGIN                                     // Alg. 2 l.7 with the indicator of R_+
    double2 h[kU], u[kU];
    ABL_FOR_K { ABL_X { h[k] = ld2(Ht, x); u[k] = ld2(U, x); } }
    ABL_FOR_K { ABL_X st2(H, x, prox0(h[k].x - u[k].x), prox0(h[k].y - u[k].y)); }
  ABL_LOOP_END
  ABL_TAIL H[n - 1] = prox0(Ht[n - 1] - U[n - 1]);
}
__global__ void k_dual(const double* __restrict__ H, const double* __restrict__ Ht, double* __restrict__ U, int64_t n) {
  ABL_LOOP_BEGIN                                     // Alg. 2 l.8
    double2 h[kU], t[kU], u[kU];
    ABL_FOR_K { ABL_X { h[k] = ld2(H, x); t[k] = ld2(Ht, x); u[k] = ld2(U, x); } }
    ABL_FOR_K { ABL_X st2(U, x, u[k].x + h[k].x - t[k].x, u[k].y + h[k].y - t[k].y); }
  ABL_LOOP_END
  ABL_TAIL U[n - 1] = U[n - 1] + H[n - 1] - Ht[n - 1];
}

__device__ __forceinline__ void block_store4(double a, double b, double c, double d, double* __restrict__ part) {
  __shared__ double red[4][kT];
  red[0][threadIdx.x] = a; red[1][threadIdx.x] = b; red[2][threadIdx.x] = c; red[3][threadIdx.x] = d;
  __syncthreads();
  for (int k = kT / 2; k > 0; k >>= 1) {
    if (threadIdx.x < k)
      for (int w = 0; w < 4; w++) red[w][threadIdx.x] += red[w][threadIdx.x + k];
    __syncthreads();
  }
  if (threadIdx.x < 4) part[blockIdx.x * 4 + threadIdx.x] = red[threadIdx.x][0];
}
__device__ __forceinline__ void acc4(double h, double ht, double h0, double u, double& r, double& s, double& nh,
                                     double& nu) {
  const double e1 = h - ht, e2 = h - h0;
  r += e1 * e1; s += e2 * e2; nh += h * h; nu += u * u;
}
// residual sums of the baseline (the norms of Alg. 2 l.9, one pass over the four matrices)
__global__ void k_resid(const double* __restrict__ H, const double* __restrict__ Ht, const double* __restrict__ H0,
                        const double* __restrict__ U, int64_t n, double* __restrict__ part) {
  double r = 0, s = 0, h = 0, u = 0;
  ABL_LOOP_BEGIN
    double2 a[kU], t[kU], z[kU], v[kU];
    ABL_FOR_K { ABL_X { a[k] = ld2(H, x); t[k] = ld2(Ht, x); z[k] = ld2(H0, x); v[k] = ld2(U, x); } }
    ABL_FOR_K {
      ABL_X {
        acc4(a[k].x, t[k].x, z[k].x, v[k].x, r, s, h, u);
        acc4(a[k].y, t[k].y, z[k].y, v[k].y, r, s, h, u);
      }
    }
  ABL_LOOP_END
  ABL_TAIL acc4(H[n - 1], Ht[n - 1], H0[n - 1], U[n - 1], r, s, h, u);
  block_store4(r, s, h, u, part);
}

// ---- fused kernels (operation fusion, Sec. 4.3.1)
// T = M + rho (H + U): reads 3 I R, writes I R (L823-829)
__global__ void k_fused_T(const double* __restrict__ M, const double* __restrict__ H, const double* __restrict__ U,
                          const double* __restrict__ consts, double* __restrict__ T, int64_t n) {
  const double rho = consts[1];
  ABL_LOOP_BEGIN
    double2 m[kU], h[kU], u[kU];
    ABL_FOR_K { ABL_X { m[k] = ld2(M, x); h[k] = ld2(H, x); u[k] = ld2(U, x); } }
    ABL_FOR_K { ABL_X st2(T, x, m[k].x + rho * (h[k].x + u[k].x), m[k].y + rho * (h[k].y + u[k].y)); }
  ABL_LOOP_END
  ABL_TAIL T[n - 1] = M[n - 1] + rho * (H[n - 1] + U[n - 1]);
}
// prox + dual + residual partials in one pass; H0 is the incoming H (no copy)
__device__ __forceinline__ void epi1(double ht, double h0, double u0, double& hn, double& un, double& r, double& s,
                                     double& nh, double& nu) {
  hn = prox0(ht - u0);
  un = u0 + hn - ht;
  acc4(hn, ht, h0, un, r, s, nh, nu);
}
__global__ void k_fused_epi(const double* __restrict__ Ht, double* __restrict__ H, double* __restrict__ U, int64_t n,
                            double* __restrict__ part) {
  double r = 0, s = 0, h = 0, u = 0;
  ABL_LOOP_BEGIN
    double2 t[kU], h0[kU], u0[kU];
    ABL_FOR_K { ABL_X { t[k] = ld2(Ht, x); h0[k] = ld2(H, x); u0[k] = ld2(U, x); } }
    ABL_FOR_K {
      ABL_X {
        double a, b, c, d;
        epi1(t[k].x, h0[k].x, u0[k].x, a, c, r, s, h, u);
        epi1(t[k].y, h0[k].y, u0[k].y, b, d, r, s, h, u);
        st2(H, x, a, b);
        st2(U, x, c, d);
      }
    }
  ABL_LOOP_END
  ABL_TAIL {
    double a, c;
    epi1(Ht[n - 1], H[n - 1], U[n - 1], a, c, r, s, h, u);
    H[n - 1] = a;
    U[n - 1] = c;
  }
  block_store4(r, s, h, u, part);
}

// fixed-order sum of the per-CTA partials of pass j -> sums[j][4]
__global__ void k_sum(const double* __restrict__ part, int nb, double* __restrict__ sums) {
  if (threadIdx.x >= 4) return;
  double s = 0.0;
  for (int b = 0; b < nb; b++) s += part[b * 4 + threadIdx.x];
  sums[threadIdx.x] = s;
}

struct Ws {
  cublasHandle_t h = nullptr;
  void* p = nullptr;
  size_t bytes = 0;
  int dev = -1;
};
thread_local Ws g_ws[64];

int ensure(Ws& w, size_t bytes) {
  if (w.bytes >= bytes) return 0;
  if (w.p) cudaFree(w.p);
  w.p = nullptr;
  w.bytes = 0;
  ACU(cudaMalloc(&w.p, bytes));
  w.bytes = bytes;
  return 0;
}

// FP64 tensor-path peak ("measure on the box the FP64 DMMA peak"):
// 8 independent m8n8k4 f64 accumulator chains per warp, no memory traffic.
__global__ void __launch_bounds__(256) k_dmma_peak(double* out, int iters) {
  const double a = threadIdx.x * 1e-3, b = threadIdx.x * 2e-3;
  double c[8][2];
#pragma unroll
  for (int t = 0; t < 8; t++) c[t][0] = c[t][1] = 0.0;
  for (int i = 0; i < iters; i++) {
#pragma unroll
    for (int t = 0; t < 8; t++)
      asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
                   : "+d"(c[t][0]), "+d"(c[t][1]) : "d"(a), "d"(b));
  }
  double s = 0.0;
#pragma unroll
  for (int t = 0; t < 8; t++) s += c[t][0] + c[t][1];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

}  // namespace

extern "C" {

const char* cstf_ablation_last_error(void) { return g_err.c_str(); }
int64_t cstf_ablation_last_calls(void) { return g_calls; }

int cstf_ablation_admm(int arm, const double* d_M, const double* d_S, double* d_H, double* d_U, int64_t I, int R,
                       int max_iter, double* stats_out, void* stream) {
  g_calls = 0;
  if (arm < CSTF_ABL_BASELINE || arm > CSTF_ABL_OF_PI) return err("unknown arm");
  if (R < 1 || R > 64 || I < 1 || max_iter < 1) return err("need R in [1, 64], I >= 1, max_iter >= 1");
  if (((uintptr_t)d_M | (uintptr_t)d_H | (uintptr_t)d_U) & 15) return err("M, H, U must be 16-byte aligned");
  const bool fuse = arm == CSTF_ABL_OF || arm == CSTF_ABL_OF_PI;
  const bool pinv = arm == CSTF_ABL_PI || arm == CSTF_ABL_OF_PI;
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  int dev = 0, sms = 0;
  ACU(cudaGetDevice(&dev));
  ACU(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
  Ws& w = g_ws[dev & 63];
  if (!w.h) {
    if (cublasCreate(&w.h) != CUBLAS_STATUS_SUCCESS) return err("cublasCreate");
  }
  ABL(cublasSetStream(w.h, st));
  ABL(cublasSetPointerMode(w.h, CUBLAS_POINTER_MODE_DEVICE));
  const int64_t n = I * R;
  const int nb = (int)std::max<int64_t>(1, std::min<int64_t>((n / 2 + kT - 1) / kT, (int64_t)sms * 16));
  // workspace: Ht, T, H0 (I x R each), L, Inv (R x R), consts[4], partials, sums, flag
  const int64_t np = (n + 1) & ~(int64_t)1;      // even offsets keep every matrix 16-byte aligned
  const size_t need = (size_t)(3 * np + 2 * R * R + 4 + nb * 4 + (size_t)max_iter * 4 + 2) * 8;
  if (ensure(w, need)) return 1;
  double* Ht = static_cast<double*>(w.p);
  double* Tb = Ht + np;
  double* H0 = Tb + np;
  double* Lc = H0 + np;
  double* Inv = Lc + R * R;
  double* cst = Inv + R * R;
  double* part = cst + 4;
  double* sums = part + (size_t)nb * 4;
  int* flag = reinterpret_cast<int*>(sums + (size_t)max_iter * 4);
  ACU(cudaFuncSetAttribute(k_chol, cudaFuncAttributeMaxDynamicSharedMemorySize, 2 * 64 * 64 * 8));
  k_chol<<<1, 128, (size_t)2 * R * R * 8, st>>>(d_S, R, pinv ? 1 : 0, Lc, Inv, cst, flag);
  LAUNCHED();
  const double* one = cst;
  const double* rho = cst + 1;
  const double* zero = cst + 2;
  // T = M + rho (H + U) goes to Tb when a DGEMM follows (not in place), else to Ht
  double* T = pinv ? Tb : Ht;
  for (int j = 0; j < max_iter; j++) {
    if (!fuse) {                                   // Alg. 2 l.5-6 as separate calls
      ACU(cudaMemcpyAsync(H0, d_H, (size_t)n * 8, cudaMemcpyDeviceToDevice, st));
      g_calls++;
      // column-major view of the row-major I x R matrices: R x I, ld = R
      ABL(cublasDgeam(w.h, CUBLAS_OP_N, CUBLAS_OP_N, R, (int)I, one, d_H, R, one, d_U, R, T, R));   // H + U
      ABL(cublasDgeam(w.h, CUBLAS_OP_N, CUBLAS_OP_N, R, (int)I, one, d_M, R, rho, T, R, T, R));     // M + rho (.)
    } else {
      k_fused_T<<<nb, kT, 0, st>>>(d_M, d_H, d_U, cst, T, n);
      LAUNCHED();
    }
    if (pinv) {                                    // H~^T = Inv T^T: one DGEMM per pass
      ABL(cublasDgemm(w.h, CUBLAS_OP_N, CUBLAS_OP_N, R, (int)I, R, one, Inv, R, T, R, zero, Ht, R));
    } else {                                       // L Y = T^T, then L^T H~^T = Y (in place)
      ABL(cublasDtrsm(w.h, CUBLAS_SIDE_LEFT, CUBLAS_FILL_MODE_LOWER, CUBLAS_OP_N, CUBLAS_DIAG_NON_UNIT, R, (int)I, one,
                      Lc, R, Ht, R));
      ABL(cublasDtrsm(w.h, CUBLAS_SIDE_LEFT, CUBLAS_FILL_MODE_LOWER, CUBLAS_OP_T, CUBLAS_DIAG_NON_UNIT, R, (int)I, one,
                      Lc, R, Ht, R));
    }
    if (!fuse) {                                   // Alg. 2 l.7-9 as separate calls
      k_prox<<<nb, kT, 0, st>>>(Ht, d_U, d_H, n);
      LAUNCHED();
      k_dual<<<nb, kT, 0, st>>>(d_H, Ht, d_U, n);
      LAUNCHED();
      k_resid<<<nb, kT, 0, st>>>(d_H, Ht, H0, d_U, n, part);
      LAUNCHED();
    } else {
      k_fused_epi<<<nb, kT, 0, st>>>(Ht, d_H, d_U, n, part);
      LAUNCHED();
    }
    k_sum<<<1, 32, 0, st>>>(part, nb, sums + (size_t)j * 4);
    LAUNCHED();
  }
  double host[6];
  int hflag = 0;
  ACU(cudaMemcpyAsync(host + 2, sums + (size_t)(max_iter - 1) * 4, 32, cudaMemcpyDeviceToHost, st));
  ACU(cudaMemcpyAsync(host + 1, cst + 1, 8, cudaMemcpyDeviceToHost, st));
  ACU(cudaMemcpyAsync(&hflag, flag, 4, cudaMemcpyDeviceToHost, st));
  ACU(cudaStreamSynchronize(st));
  if (hflag) return err("S + rho I is not positive definite");
  host[0] = max_iter;
  if (stats_out)
    for (int k = 0; k < 6; k++) stats_out[k] = host[k];
  return 0;
}

double cstf_ablation_fp64_peak(void* stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  int dev = 0, sms = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess)
    return -1.0;
  const int grid = sms * 8, bs = 256, iters = 4096;
  double* out = nullptr;
  cudaEvent_t e0, e1;
  if (cudaMalloc(&out, (size_t)grid * bs * 8) != cudaSuccess) return -1.0;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  k_dmma_peak<<<grid, bs, 0, st>>>(out, 64);                 // warm-up (clocks up)
  float best = 1e30f;
  for (int r = 0; r < 3; r++) {
    cudaEventRecord(e0, st);
    k_dmma_peak<<<grid, bs, 0, st>>>(out, iters);
    cudaEventRecord(e1, st);
    cudaEventSynchronize(e1);
    float ms = 0.f;
    cudaEventElapsedTime(&ms, e0, e1);
    best = std::min(best, ms);
  }
  const cudaError_t e = cudaGetLastError();
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  cudaFree(out);
  if (e != cudaSuccess || best <= 0.f) return -1.0;
  const double flops = 2.0 * 256 * 8 * (double)iters * grid * (bs / 32);    // 8 chains x 512 flops per warp
  return flops / (best * 1e-3) / 1e12;
}

}  // extern "C"
