// Dense R x R / I x R kernels of the hot path:
//   a1 S = *_{k!=n} G^(k)            Alg. 1 l.8 (L494)
//   a3 rho = tr(S)/R                 Alg. 2/3 l.2 (L558, L642)
//   a4 S + rho I = L L^T, Inv = (L L^T)^{-1}   Alg. 3 l.3-4 (L644-646), pre-inversion Sec. 4.3.2
//   a6 normalize, a7 Gram            Alg. 1 l.11-12 (L499, L501)
//   a8 fit                           reading D12
// All reductions use a fixed grid and fixed summation order (deterministic).
#include "internal.h"

namespace cstf {
namespace {

constexpr int kGramThreads = 256;
constexpr int kGramTile = 32;   // rows staged per step
constexpr int kGramMaxP = 3;    // pairs per thread (R = 128: 528 pairs / 256 threads)

int gram_blocks(int64_t I) {
  int64_t b = (I + 511) / 512;
  int cap = device_info().sms * 2;
  if (b > cap) b = cap;
  return (int)(b < 1 ? 1 : b);
}

// Per block: partial of H^T H over its row tiles (grid-stride by tile).  The
// R x R result is cut into 4x4 register tiles; only tile pairs (A <= B) of the
// upper triangle are computed.  When there are fewer pairs than threads,
// several thread groups split the rows of a staged tile and are summed at the
// end in group order (deterministic).  part layout: [block][pair][16].
__global__ void __launch_bounds__(kGramThreads) k_gram_partial(const double* __restrict__ H, int64_t I,
                                                               int R, double* __restrict__ part) {
  extern __shared__ double sm[];
  const int RP = (R + 3) & ~3;
  const int nb4 = RP / 4;
  const int npairs = nb4 * (nb4 + 1) / 2;
  const int ngroups = npairs >= kGramThreads ? 1 : kGramThreads / npairs;
  double* tile = sm;                              // [kGramTile][RP]
  double* red = sm + kGramTile * RP;              // [ngroups][npairs][16] (only if ngroups > 1)
  const int t = threadIdx.x;
  const int g = (ngroups > 1) ? t / npairs : 0;
  int pa[kGramMaxP], pb[kGramMaxP];
  bool pact[kGramMaxP];
#pragma unroll
  for (int s = 0; s < kGramMaxP; s++) {
    const int p = (ngroups > 1) ? t % npairs : t + s * kGramThreads;
    pact[s] = (ngroups > 1) ? (s == 0 && t < npairs * ngroups) : (p < npairs);
    int a = 0, rem = pact[s] ? p : 0;
    while (rem >= nb4 - a) { rem -= nb4 - a; a++; }
    pa[s] = a; pb[s] = a + rem;
  }
  double acc[kGramMaxP][16];
#pragma unroll
  for (int s = 0; s < kGramMaxP; s++)
#pragma unroll
    for (int e = 0; e < 16; e++) acc[s][e] = 0.0;
  const int64_t ntiles = (I + kGramTile - 1) / kGramTile;
  for (int64_t tl = blockIdx.x; tl < ntiles; tl += gridDim.x) {
    const int64_t r0 = tl * kGramTile;
    const int rows = (int)min((int64_t)kGramTile, I - r0);
    for (int x = t; x < kGramTile * RP; x += blockDim.x) {
      const int r = x / RP, c = x % RP;
      tile[x] = (r < rows && c < R) ? H[(r0 + r) * R + c] : 0.0;
    }
    __syncthreads();
#pragma unroll
    for (int s = 0; s < kGramMaxP; s++) {
      if (!pact[s]) continue;
      const double* ta = tile + 4 * pa[s];
      const double* tb = tile + 4 * pb[s];
      for (int r = g; r < kGramTile; r += ngroups) {
        const double2 a01 = *reinterpret_cast<const double2*>(ta + r * RP);
        const double2 a23 = *reinterpret_cast<const double2*>(ta + r * RP + 2);
        const double2 b01 = *reinterpret_cast<const double2*>(tb + r * RP);
        const double2 b23 = *reinterpret_cast<const double2*>(tb + r * RP + 2);
        const double av[4] = {a01.x, a01.y, a23.x, a23.y};
        const double bv[4] = {b01.x, b01.y, b23.x, b23.y};
#pragma unroll
        for (int i = 0; i < 4; i++)
#pragma unroll
          for (int j = 0; j < 4; j++) acc[s][i * 4 + j] = fma(av[i], bv[j], acc[s][i * 4 + j]);
      }
    }
    __syncthreads();
  }
  if (ngroups > 1) {
    if (pact[0])
#pragma unroll
      for (int e = 0; e < 16; e++) red[((size_t)g * npairs + (t % npairs)) * 16 + e] = acc[0][e];
    __syncthreads();
    for (int x = t; x < npairs * 16; x += blockDim.x) {
      double v = 0.0;
      for (int gg = 0; gg < ngroups; gg++) v += red[(size_t)gg * npairs * 16 + x];
      part[(int64_t)blockIdx.x * npairs * 16 + x] = v;
    }
  } else {
#pragma unroll
    for (int s = 0; s < kGramMaxP; s++) {
      if (!pact[s]) continue;
      const int p = t + s * kGramThreads;
#pragma unroll
      for (int e = 0; e < 16; e++) part[((int64_t)blockIdx.x * npairs + p) * 16 + e] = acc[s][e];
    }
  }
}

// G (full R x R) = sum over blocks in block order, mirrored from the tile pairs.
__global__ void k_gram_sum(const double* __restrict__ part, int nb, int R, double* __restrict__ G) {
  const int RP = (R + 3) & ~3;
  const int nb4 = RP / 4;
  const int npairs = nb4 * (nb4 + 1) / 2;
  for (int x = blockIdx.x * blockDim.x + threadIdx.x; x < npairs * 16; x += gridDim.x * blockDim.x) {
    const int p = x / 16, e = x % 16;
    int A = 0, rem = p;
    while (rem >= nb4 - A) { rem -= nb4 - A; A++; }
    const int B = A + rem;
    const int a = 4 * A + e / 4, b = 4 * B + e % 4;
    if (a >= R || b >= R) continue;
    if (A == B && a > b) continue;   // diagonal tile: take the upper triangle, mirror it
    double s = 0.0;
    for (int k = 0; k < nb; k++) s += part[(int64_t)k * npairs * 16 + x];
    G[a * R + b] = s;
    G[b * R + a] = s;
  }
}

size_t gram_smem(int R) {
  const int RP = (R + 3) & ~3;
  const int nb4 = RP / 4;
  const int npairs = nb4 * (nb4 + 1) / 2;
  const int ngroups = npairs >= kGramThreads ? 1 : kGramThreads / npairs;
  return (size_t)kGramTile * RP * 8 + (ngroups > 1 ? (size_t)ngroups * npairs * 16 * 8 : 0);
}

// lam_r = sqrt(G_rr); G <- D^-1 G D^-1 (entries of zero columns stay 0, D8)
__global__ void k_gram_normalize(double* __restrict__ G, int R, double* __restrict__ lam) {
  __shared__ double sl[128];
  for (int a = threadIdx.x; a < R; a += blockDim.x) {
    sl[a] = sqrt(G[a * R + a]);
    lam[a] = sl[a];
  }
  __syncthreads();
  for (int e = threadIdx.x; e < R * R; e += blockDim.x) {
    const int a = e / R, b = e % R;
    G[e] = (sl[a] > 0.0 && sl[b] > 0.0) ? G[e] / sl[a] / sl[b] : 0.0;
  }
}

// x / l for l > 0 from the rounded reciprocal r = 1/l: q = x r, e = x - q l (exact by
// fma), q + e r is the IEEE quotient (Markstein's correction: r is the correctly rounded
// reciprocal and nothing over- or underflows in the guarded range; bitwise equal to the
// division, tests/test_gpu_parity.py test_normalize_division_exact).  Outside the range
// the division itself.
__device__ __forceinline__ double div_by(double x, double l, double r) {
  const double ax = fabs(x);
  if (l >= 0x1p-900 && l <= 0x1p900 && (ax == 0.0 || (ax >= 0x1p-900 && ax <= 0x1p900))) {
    const double q = x * r;
    return fma(fma(-q, l, x), r, q);
  }
  return x / l;
}

// Even R, 16-byte aligned H: pairs of columns (a pair never straddles a row), 4 pairs in
// flight per thread, one wave of resident CTAs (launch_scale); the column factors and their
// reciprocals in shared memory.  (The scalar kernel below ran at ~2.5 TB/s: 2,368 CTAs in
// 3.2 waves of 740 resident, plus an FP64 division sequence per element.)
__global__ void k_scale_cols2(double2* __restrict__ H, int64_t I, int R, const double* __restrict__ lam,
                              int divide) {
  constexpr int U = 4;
  __shared__ double sl[128], sr[128];
  for (int c = threadIdx.x; c < R; c += blockDim.x) {
    sl[c] = lam[c];
    sr[c] = (divide && lam[c] > 0.0) ? 1.0 / lam[c] : 0.0;
  }
  __syncthreads();
  const int R2 = R / 2;
  const int64_t n = I * R2;
  const int64_t x0 = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  const int64_t step = (int64_t)gridDim.x * blockDim.x;
  const int dstep = (int)(step % R2);          // pair column advances by a constant
  int col = (int)(x0 % R2);
  for (int64_t x = x0; x < n; x += U * step) {
    double2 v[U];
    int cc[U];
#pragma unroll
    for (int k = 0; k < U; k++) {
      cc[k] = col;
      col += dstep;
      if (col >= R2) col -= R2;
      if (x + k * step < n) v[k] = __ldcs(H + x + k * step);
    }
#pragma unroll
    for (int k = 0; k < U; k++) {
      if (x + k * step >= n) break;
      const int c = 2 * cc[k];
      const double l0 = sl[c], l1 = sl[c + 1];
      double2 o = v[k];
      if (divide) {
        if (l0 > 0.0) o.x = div_by(v[k].x, l0, sr[c]);
        if (l1 > 0.0) o.y = div_by(v[k].y, l1, sr[c + 1]);
      } else {
        o.x = v[k].x * l0;
        o.y = v[k].y * l1;
      }
      __stcs(H + x + k * step, o);
    }
  }
}

__global__ void k_scale_cols(double* __restrict__ H, int64_t I, int R, const double* __restrict__ lam,
                             int divide) {
  // 4 elements per thread and iteration, all loaded before any is scaled (one load
  // in flight per thread left this streaming pass at ~2.5 TB/s)
  constexpr int U = 4;
  const int64_t n = I * R;
  const int64_t x0 = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  const int64_t step = (int64_t)gridDim.x * blockDim.x;
  const int dstep = (int)(step % R);          // column advances by a constant: no per-element modulo
  int col = (int)(x0 % R);
  for (int64_t x = x0; x < n; x += U * step) {
    double v[U];
    int c[U];
#pragma unroll
    for (int k = 0; k < U; k++) {
      c[k] = col;
      col += dstep;
      if (col >= R) col -= R;
      if (x + k * step < n) v[k] = H[x + k * step];
    }
#pragma unroll
    for (int k = 0; k < U; k++) {
      if (x + k * step >= n) break;
      const double l = lam[c[k]];
      if (divide) {
        if (l > 0.0) H[x + k * step] = v[k] / l;
      } else {
        H[x + k * step] = v[k] * l;
      }
    }
  }
}

__global__ void k_fill(double* __restrict__ d, int64_t n, double v) {
  for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < n; x += (int64_t)gridDim.x * blockDim.x)
    d[x] = v;
}

// One CTA.  S (from d_S or Hadamard of the Grams except `skip`, increasing k),
// rho = tr(S)/R (or rho_in > 0), right-looking Cholesky of S + rho I in shared
// memory, L^-1 by forward substitution on all columns at once, Inv = L^-T L^-1
// (pre-inversion, Sec. 4.3.2).  kappa(S + rho I) <= R + 1 (pin P5) keeps the
// explicit inverse accurate.
__global__ void k_chol_inverse(const double* __restrict__ S_in, const double* __restrict__ grams,
                               int N, int skip, int R, double rho_in, double* __restrict__ Linv,
                               double* __restrict__ Inv, double* __restrict__ scal, int* flag,
                               const double* __restrict__ lam, double* __restrict__ colscale,
                               double* __restrict__ S_out) {
  if (lam) {
    for (int r = threadIdx.x; r < R; r += blockDim.x) {
      double ms = 1.0;
      for (int k = 0; k < N; k++) {
        if (k == skip) continue;
        const double l = lam[k * R + r];
        ms = (l > 0.0) ? ms / l : 0.0;
      }
      colscale[r] = ms;
      const double ls = lam[skip * R + r];
      colscale[R + r] = (ls > 0.0) ? 1.0 / ls : 0.0;
    }
  }
  extern __shared__ double L[];  // [R][R]: A, then L in the lower triangle; then [R][R] L^-1 if it fits
  __shared__ double s_rho;
  if (R <= 64) Linv = L + R * R;   // shared-memory copy of L^-1 (latency-bound loops below)
  __shared__ int s_bad;
  const int RR = R * R;
  for (int e = threadIdx.x; e < RR; e += blockDim.x) {
    double v;
    if (grams) {
      v = 1.0;
      bool first = true;
      for (int k = 0; k < N; k++) {
        if (k == skip) continue;
        const double g = grams[(int64_t)k * RR + e];
        v = first ? g : __dmul_rn(v, g);
        first = false;
      }
    } else {
      v = S_in[e];
    }
    L[e] = v;
    if (S_out) S_out[e] = v;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    double rho = rho_in;
    if (!(rho_in > 0.0)) {
      double tr = 0.0;
      for (int a = 0; a < R; a++) tr = __dadd_rn(tr, L[a * R + a]);
      rho = tr / R;
    }
    s_rho = rho;
    s_bad = !(rho > 0.0);
    scal[0] = rho;
  }
  __syncthreads();
  const double rho = s_rho;
  for (int a = threadIdx.x; a < R; a += blockDim.x) L[a * R + a] = __dadd_rn(L[a * R + a], rho);
  __syncthreads();
  // right-looking Cholesky: step j scales column j and updates the trailing
  // lower triangle in parallel (two barriers per step)
  for (int j = 0; j < R; j++) {
    if (threadIdx.x == 0) {
      const double s = L[j * R + j];
      if (!(s > 0.0)) s_bad = 1;
      L[j * R + j] = sqrt(s > 0.0 ? s : 1.0);
    }
    __syncthreads();
    const double d = L[j * R + j];
    for (int i = j + 1 + threadIdx.x; i < R; i += blockDim.x) L[i * R + j] = L[i * R + j] / d;
    __syncthreads();
    const int m = R - j - 1;                      // trailing block (j+1..R-1)^2, lower part
    for (int e = threadIdx.x; e < m * m; e += blockDim.x) {
      const int i = j + 1 + e / m, k = j + 1 + e % m;
      if (k <= i) L[i * R + k] = fma(-L[i * R + j], L[k * R + j], L[i * R + k]);
    }
    __syncthreads();
  }
  // L^-1 by forward substitution on all columns at once: step a fixes row a
  // of L^-1, then eliminates it from the rows below
  for (int e = threadIdx.x; e < R * R; e += blockDim.x) {
    const int i = e / R, c = e % R;
    Linv[e] = (i == c) ? 1.0 : 0.0;
  }
  __syncthreads();
  for (int a = 0; a < R; a++) {
    const double inv_d = 1.0 / L[a * R + a];
    for (int c = threadIdx.x; c <= a; c += blockDim.x) Linv[a * R + c] *= inv_d;
    __syncthreads();
    const int m = R - a - 1;
    for (int e = threadIdx.x; e < m * (a + 1); e += blockDim.x) {
      const int i = a + 1 + e / (a + 1), c = e % (a + 1);
      Linv[i * R + c] = fma(-L[i * R + a], Linv[a * R + c], Linv[i * R + c]);
    }
    __syncthreads();
  }
  // Inv[a][b] = sum_{k >= max(a,b)} Linv[k][a] Linv[k][b]   (computed for a <= b, mirrored)
  for (int e = threadIdx.x; e < RR; e += blockDim.x) {
    const int a = e / R, b = e % R;
    if (a > b) continue;
    double s = 0.0;
    for (int k = b; k < R; k++) s = fma(Linv[k * R + a], Linv[k * R + b], s);
    Inv[a * R + b] = s;
    Inv[b * R + a] = s;
  }
  if (threadIdx.x == 0 && s_bad) atomicOr(flag, 1);
}

// fit: per block partial of sum_i sum_r M_ir H_ir lam_r
__global__ void __launch_bounds__(256) k_fit_partial(const double* __restrict__ M, const double* __restrict__ H,
                                                     const double* __restrict__ colw, int64_t I, int R,
                                                     double* __restrict__ part) {
  __shared__ double sh[256];
  const int64_t n = I * R;
  double acc = 0.0;
  const int64_t x0 = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  const int64_t step = (int64_t)gridDim.x * blockDim.x;
  const int dstep = (int)(step % R);
  int col = (int)(x0 % R);
  for (int64_t x = x0; x < n; x += step) {
    acc = fma(M[x] * H[x], colw[col], acc);
    col += dstep;
    if (col >= R) col -= R;
  }
  sh[threadIdx.x] = acc;
  __syncthreads();
  for (int s = 128; s > 0; s >>= 1) {
    if (threadIdx.x < s) sh[threadIdx.x] += sh[threadIdx.x + s];
    __syncthreads();
  }
  if (threadIdx.x == 0) part[blockIdx.x] = sh[0];
}

__global__ void k_fit_sum(const double* __restrict__ part, int nb, double* __restrict__ out) {
  if (threadIdx.x == 0 && blockIdx.x == 0) {
    double s = 0.0;
    for (int b = 0; b < nb; b++) s += part[b];
    out[1] = s;
  }
}

__global__ void k_fit_final(double normX2, const double* __restrict__ lam, const double* __restrict__ grams,
                            int N, int R, double* __restrict__ out, int* flag) {
  __shared__ double sh[256];
  double acc = 0.0;
  for (int e = threadIdx.x; e < R * R; e += blockDim.x) {
    const int a = e / R, b = e % R;
    double g = 1.0;
    for (int k = 0; k < N; k++) g *= grams[(int64_t)k * R * R + e];
    acc = fma(lam[a] * lam[b], g, acc);
  }
  sh[threadIdx.x] = acc;
  __syncthreads();
  for (int s = blockDim.x / 2; s > 0; s >>= 1) {
    if (threadIdx.x < s) sh[threadIdx.x] += sh[threadIdx.x + s];
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    const double xhat = sh[0];
    double res2 = normX2 + xhat - 2.0 * out[1];
    if (res2 < 0.0) res2 = 0.0;
    const double f = 1.0 - sqrt(res2) / sqrt(normX2);
    out[0] = f;
    if (!isfinite(f)) atomicOr(flag, 2);
  }
}

struct Workspace {
  DevBuf part, linv;
};
Workspace& ws() {
  static thread_local Workspace w[64];
  int dev = 0;
  cudaGetDevice(&dev);
  return w[dev & 63];
}

}  // namespace

void release_dense_ws() {
  Workspace& w = ws();
  w.part.release();
  w.linv.release();
}

cstf_status fill(double* d, int64_t n, double v, cudaStream_t st) {
  if (n <= 0) return CSTF_OK;
  int g = (int)std::min<int64_t>((n + 255) / 256, (int64_t)device_info().sms * 16);
  k_fill<<<g, 256, 0, st>>>(d, n, v);
  CSTF_LAUNCHED();
  return CSTF_OK;
}

cstf_status scale_rows_by_cols(double* d_H, int64_t I, int R, const double* d_lam, int divide,
                               cudaStream_t st) {
  if (I * R == 0) return CSTF_OK;
  if (R % 2 == 0 && R <= 128 && (reinterpret_cast<uintptr_t>(d_H) & 15) == 0) {
    static int per_sm = 0;
    if (!per_sm) {
      CSTF_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_scale_cols2, 256, 0));
      if (per_sm < 1) per_sm = 1;
    }
    const int g = (int)std::min<int64_t>((I * (R / 2) + 255) / 256, (int64_t)device_info().sms * per_sm);
    k_scale_cols2<<<g, 256, 0, st>>>(reinterpret_cast<double2*>(d_H), I, R, d_lam, divide);
    CSTF_LAUNCHED();
    return CSTF_OK;
  }
  int g = (int)std::min<int64_t>((I * R + 255) / 256, (int64_t)device_info().sms * 16);
  k_scale_cols<<<g, 256, 0, st>>>(d_H, I, R, d_lam, divide);
  CSTF_LAUNCHED();
  return CSTF_OK;
}

cstf_status gram_raw(const double* d_H, int64_t I, int R, double* d_G, cudaStream_t st) {
  cstf_status gs = CSTF_OK;
  if (gram_dmma(d_H, I, R, d_G, st, &gs)) return gs;      // R <= 64: FP64 tensor path (admm.cu)
  const int nb = gram_blocks(I);
  const int nb4 = ((R + 3) & ~3) / 4;
  const int E = nb4 * (nb4 + 1) / 2 * 16;
  Workspace& w = ws();
  CSTF_TRY(w.part.ensure((size_t)nb * E * 8));
  const size_t smem = gram_smem(R);
  static bool attr_set = false;
  if (!attr_set) {
    CSTF_CUDA(cudaFuncSetAttribute(k_gram_partial, cudaFuncAttributeMaxDynamicSharedMemorySize, 96 * 1024));
    attr_set = true;
  }
  k_gram_partial<<<nb, kGramThreads, smem, st>>>(d_H, I, R, w.part.as<double>());
  CSTF_LAUNCHED();
  k_gram_sum<<<(E + 255) / 256, 256, 0, st>>>(w.part.as<double>(), nb, R, d_G);
  CSTF_LAUNCHED();
  return CSTF_OK;
}

cstf_status normalize_from_gram(double* d_H, int64_t I, int R, double* d_G, double* d_lam,
                                cudaStream_t st) {
  k_gram_normalize<<<1, 1024, 0, st>>>(d_G, R, d_lam);
  CSTF_LAUNCHED();
  return scale_rows_by_cols(d_H, I, R, d_lam, 1, st);
}

cstf_status gram_normalize(double* d_H, int64_t I, int R, double* d_G, double* d_lam,
                           const cstf_comm* comm, cudaStream_t st, int64_t* launches) {
  CSTF_TRY(gram_raw(d_H, I, R, d_G, st));
  CSTF_TRY(comm_allreduce_f64(comm, d_G, (size_t)R * R, st));
  int64_t nl = 2;
  if (d_lam) {
    CSTF_TRY(normalize_from_gram(d_H, I, R, d_G, d_lam, st));
    nl += (I * R > 0) ? 2 : 1;
  }
  if (launches) *launches += nl;
  return CSTF_OK;
}

cstf_status gram_to_lambda(double* d_G, int R, double* d_lam, cudaStream_t st) {
  k_gram_normalize<<<1, 1024, 0, st>>>(d_G, R, d_lam);
  CSTF_LAUNCHED();
  return CSTF_OK;
}

cstf_status chol_inverse(const double* d_S, const double* d_grams, int N, int skip, int R,
                         double rho_in, double* d_inv, double* d_scal, int* d_flag,
                         cudaStream_t st, const double* d_lam, double* d_colscale, double* d_S_out) {
  Workspace& w = ws();
  CSTF_TRY(w.linv.ensure((size_t)R * R * 8));
  const size_t smem = (size_t)R * R * 8 * (R <= 64 ? 2 : 1);
  static bool attr_set = false;
  if (!attr_set) {
    CSTF_CUDA(cudaFuncSetAttribute(k_chol_inverse, cudaFuncAttributeMaxDynamicSharedMemorySize, 128 * 1024));
    attr_set = true;
  }
  k_chol_inverse<<<1, 256, smem, st>>>(d_S, d_grams, N, skip, R, rho_in, w.linv.as<double>(), d_inv,
                                       d_scal, d_flag, d_lam, d_colscale, d_S_out);
  CSTF_LAUNCHED();
  return CSTF_OK;
}

cstf_status fit(double normX2, int64_t I, int R, const double* d_M, const double* d_H,
                const double* d_colw, const double* d_lam, const double* d_grams, int N,
                double* d_part, double* d_out, int* d_flag, const cstf_comm* comm, cudaStream_t st) {
  const int nb = 256;
  k_fit_partial<<<nb, 256, 0, st>>>(d_M, d_H, d_colw, I, R, d_part);
  CSTF_LAUNCHED();
  k_fit_sum<<<1, 32, 0, st>>>(d_part, nb, d_out);
  CSTF_LAUNCHED();
  CSTF_TRY(comm_allreduce_f64(comm, d_out + 1, 1, st));
  k_fit_final<<<1, 256, 0, st>>>(normX2, d_lam, d_grams, N, R, d_out, d_flag);
  CSTF_LAUNCHED();
  return CSTF_OK;
}

}  // namespace cstf
