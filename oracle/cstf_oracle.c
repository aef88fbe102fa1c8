/* oracle/cstf_oracle.c -- plain, slow, obviously-correct FP64 CPU oracle for
 * constrained sparse tensor factorisation with AO-ADMM (Soh et al., ICPP'24).
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference leg may load this library.  It
 * shares no code, header, table or helper with the CUDA path
 * (paper_conf_icpp_sohksc24_b200/) and never sees its outputs.
 *
 * Every function follows the paper step by step, in its order and notation:
 *   O1 oracle_coalesce      canonical nonzero order (D14, D20)
 *   O2 oracle_mttkrp        Fig. 2: m_i,: += x_ijk (b_j,: * c_k,:)
 *   O3 oracle_gram          Alg. 1 l.4/l.12 (L484, L501): G = H^T H
 *   O4 oracle_hadamard_except Alg. 1 l.8 (L494): S = *_{k!=n} G^(k)
 *   O5/O6 oracle_cholesky   Alg. 2 l.2-3 (L558-560): rho = tr(S)/R, S + rho I = L L^T
 *   O7 oracle_admm          Alg. 2 l.4-9 (L562-572), triangular solves (NOT the
 *                           pre-inverted Alg. 3: this checks pre-inversion independently)
 *   O8 oracle_normalize     Alg. 1 l.11 (L499), column 2-norm (reading D7)
 *   O10 oracle_fit          reading D12 (the paper defines no fit)
 *   O9/O11 oracle_factorize Alg. 1 (L476-506) with readings D4, D6, D11, D13
 * Readings D1-D20 are listed in DESIGN.md.
 *
 * Parity status: every function above is pinned (DESIGN.md "Oracle pins",
 * tests/test_oracle_pins.py); none is "parity unpinned".  The summation order
 * inside MTTKRP, Gram and the residual sums differs from the GPU's (U1): a
 * rounding-order difference between two pinned implementations, bounded by
 * the tolerances in tests/, not a function without a pin.
 *
 * Determinism: every reduction uses fixed 4096-row blocks summed in block
 * order, so results are bitwise identical for any OMP_NUM_THREADS (pin P11).
 * Compiled with -ffp-contract=off: no FMA contraction, plain IEEE FP64.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <time.h>

#define ORC_OK 0
#define ORC_EINVAL 1
#define ORC_ENOMEM 3
#define ORC_NOT_SPD 6
#define ORC_NUMERIC 7
#define BLK 4096

#define PROX_NONNEG 0   /* indicator of R_+ : max(0, x), L835-839 */
#define PROX_IDENTITY 1 /* unconstrained (pin P10: reduces to CP-ALS, L360-368) */
#define PROX_L1 2       /* r(H) = alpha ||H||_1: soft threshold at alpha/rho (L540-541, L615-619) */
#define PROX_NONNEG_L1 3 /* r(H) = alpha ||H||_1 + indicator(R_+): max(0, x - alpha/rho) */
#define PROX_BOX 4      /* indicator of the box [0, alpha] (alpha > 0): the projection min(max(x, 0), alpha)
                           (reading D25; SURVEY f3 "box", L540-541 / L615-619: any element-wise operator) */

/* Alg. 2 l.7: argmin_h r(h) + rho/2 (h - x)^2 for the element-wise regularisers above
 * (tau = alpha / rho for the L1 thresholds; hi = alpha for the box) */
static double prox_apply(int prox, double x, double tau, double hi) {
  switch (prox) {
    case PROX_IDENTITY: return x;
    case PROX_L1: return x > tau ? x - tau : (x < -tau ? x + tau : 0.0);
    case PROX_NONNEG_L1: return x > tau ? x - tau : 0.0;
    case PROX_BOX: return x > 0.0 ? (x < hi ? x : hi) : 0.0;
    default: return x > 0.0 ? x : 0.0;
  }
}

/* Thread count of the OpenMP regions (infrastructure, no arithmetic): torchrun sets
 * OMP_NUM_THREADS=1 in every rank, so the bench's rank 0 sets the count it reports. */
#include <omp.h>
void oracle_set_threads(int n) { if (n > 0) omp_set_num_threads(n); }
int oracle_threads(void) { return omp_get_max_threads(); }

static double now_ms(void) {
  struct timespec ts; clock_gettime(CLOCK_MONOTONIC, &ts);
  return ts.tv_sec * 1e3 + ts.tv_nsec * 1e-6;
}

/* ---------------- canonical checksum (definition shared by contract, not code) ----
 * hash = sum_p mix(p, idx_0..idx_{N-1}, bits(val)) mod 2^64 over canonical order. */
static uint64_t mix64(uint64_t z) {
  z ^= z >> 30; z *= 0xBF58476D1CE4E5B9ULL;
  z ^= z >> 27; z *= 0x94D049BB133111EBULL;
  z ^= z >> 31; return z;
}
static uint64_t entry_hash(int64_t p, int N, const int32_t* const* idx, const double* vals) {
  uint64_t z = (uint64_t)p + 1;
  for (int n = 0; n < N; n++) z = mix64(z ^ ((uint64_t)(uint32_t)idx[n][p] + (uint64_t)(n + 1) * 0x9E3779B97F4A7C15ULL));
  uint64_t vb; memcpy(&vb, &vals[p], 8);
  return mix64(z ^ vb);
}

/* ---------------- O1: coalesce ----------------------------------------------------
 * Lexicographic order by (i_1, ..., i_N); duplicates summed left to right in
 * input order; explicit zeros kept; normX2 = sum v^2 (reading D14).
 * Implemented as a stable LSD counting sort, last mode first.
 * Returns the coalesced nnz, or -1 (EINVAL: index out of range / bad args). */
static void counting_sort_stable(int64_t nnz, int64_t dim, const int32_t* key,
                                 const int64_t* in, int64_t* out, int64_t* cnt /* dim+1 */) {
  memset(cnt, 0, (size_t)(dim + 1) * sizeof(int64_t));
  for (int64_t p = 0; p < nnz; p++) cnt[key[in[p]] + 1]++;
  for (int64_t i = 0; i < dim; i++) cnt[i + 1] += cnt[i];
  for (int64_t p = 0; p < nnz; p++) out[cnt[key[in[p]]]++] = in[p];
}

int64_t oracle_coalesce(int N, const int64_t* dims, int64_t nnz, const int32_t* const* idx,
                        const double* vals, int32_t* const* out_idx, double* out_vals,
                        double* normX2, uint64_t* hash) {
  if (N < 2 || N > 8 || nnz < 0) return -1;
  int64_t maxdim = 0;
  for (int n = 0; n < N; n++) {
    if (dims[n] < 1 || dims[n] > 2147483647LL) return -1;
    if (dims[n] > maxdim) maxdim = dims[n];
  }
  for (int n = 0; n < N; n++)
    for (int64_t p = 0; p < nnz; p++)
      if (idx[n][p] < 0 || idx[n][p] >= dims[n]) return -1;
  int64_t* a = (int64_t*)malloc((size_t)(nnz > 0 ? nnz : 1) * sizeof(int64_t));
  int64_t* b = (int64_t*)malloc((size_t)(nnz > 0 ? nnz : 1) * sizeof(int64_t));
  int64_t* cnt = (int64_t*)malloc((size_t)(maxdim + 1) * sizeof(int64_t));
  if (!a || !b || !cnt) { free(a); free(b); free(cnt); return -1; }
  for (int64_t p = 0; p < nnz; p++) a[p] = p;
  for (int n = N - 1; n >= 0; n--) {
    counting_sort_stable(nnz, dims[n], idx[n], a, b, cnt);
    int64_t* t = a; a = b; b = t;
  }
  int64_t q = -1;
  for (int64_t p = 0; p < nnz; p++) {
    int64_t src = a[p];
    int same = (q >= 0);
    for (int n = 0; n < N && same; n++) same = (idx[n][src] == out_idx[n][q]);
    if (same) {
      out_vals[q] = out_vals[q] + vals[src];
    } else {
      q++;
      for (int n = 0; n < N; n++) out_idx[n][q] = idx[n][src];
      out_vals[q] = vals[src];
    }
  }
  int64_t nout = q + 1;
  double s = 0.0;
  uint64_t h = 0;
  for (int64_t p = 0; p < nout; p++) {
    s = s + out_vals[p] * out_vals[p];
    h += entry_hash(p, N, (const int32_t* const*)out_idx, out_vals);
  }
  if (normX2) *normX2 = s;
  if (hash) *hash = h;
  free(a); free(b); free(cnt);
  return nout;
}

/* Checksum of arrays already in canonical order (used by tests on host copies). */
uint64_t oracle_canonical_hash(int N, int64_t nnz, const int32_t* const* idx, const double* vals) {
  uint64_t h = 0;
  for (int64_t p = 0; p < nnz; p++) h += entry_hash(p, N, idx, vals);
  return h;
}

/* ---------------- O2: MTTKRP (Fig. 2) -------------------------------------
 * For every row i of mode `mode`, in increasing order, and each of its
 * nonzeros in canonical order:  w = *_{k != mode} H^(k)[i_k, :]  (Hadamard,
 * increasing k), then m_i += x * w.  Rows without nonzeros are 0.
 * Input must be in canonical (coalesced) order. */
int oracle_mttkrp(int N, const int64_t* dims, int64_t nnz, const int32_t* const* cidx,
                  const double* cvals, int mode, int R, const double* const* H, double* M) {
  if (mode < 0 || mode >= N || R < 1) return ORC_EINVAL;
  int64_t I = dims[mode];
  int64_t* rowptr = (int64_t*)calloc((size_t)(I + 1), sizeof(int64_t));
  int64_t* pos = (int64_t*)malloc((size_t)(nnz > 0 ? nnz : 1) * sizeof(int64_t));
  if (!rowptr || !pos) { free(rowptr); free(pos); return ORC_ENOMEM; }
  for (int64_t p = 0; p < nnz; p++) rowptr[cidx[mode][p] + 1]++;
  for (int64_t i = 0; i < I; i++) rowptr[i + 1] += rowptr[i];
  {
    int64_t* fill = (int64_t*)malloc((size_t)(I + 1) * sizeof(int64_t));
    memcpy(fill, rowptr, (size_t)(I + 1) * sizeof(int64_t));
    for (int64_t p = 0; p < nnz; p++) pos[fill[cidx[mode][p]]++] = p;   /* stable */
    free(fill);
  }
#pragma omp parallel for schedule(dynamic, 64)
  for (int64_t i = 0; i < I; i++) {
    double* m = M + i * R;
    for (int r = 0; r < R; r++) m[r] = 0.0;
    for (int64_t q = rowptr[i]; q < rowptr[i + 1]; q++) {
      int64_t p = pos[q];
      double x = cvals[p];
      for (int r = 0; r < R; r++) {
        double w = 1.0;
        int first = 1;
        for (int k = 0; k < N; k++) {
          if (k == mode) continue;
          double hv = H[k][(int64_t)cidx[k][p] * R + r];
          w = first ? hv : w * hv;
          first = 0;
        }
        m[r] = m[r] + x * w;
      }
    }
  }
  free(rowptr); free(pos);
  return ORC_OK;
}

/* Same definition for a sample of rows only (full-size parity on sampled outputs):
 * one pass over the canonical nonzeros, accumulating rows listed in `rows`. */
int oracle_mttkrp_rows(int N, const int64_t* dims, int64_t nnz, const int32_t* const* cidx,
                       const double* cvals, int mode, int R, const double* const* H,
                       int64_t nrows, const int64_t* rows, double* Mrows) {
  if (mode < 0 || mode >= N || R < 1) return ORC_EINVAL;
  int64_t I = dims[mode];
  int64_t* slot = (int64_t*)malloc((size_t)I * sizeof(int64_t));
  if (!slot) return ORC_ENOMEM;
  for (int64_t i = 0; i < I; i++) slot[i] = -1;
  for (int64_t s = 0; s < nrows; s++) {
    if (rows[s] < 0 || rows[s] >= I) { free(slot); return ORC_EINVAL; }
    slot[rows[s]] = s;
  }
  memset(Mrows, 0, (size_t)(nrows * R) * sizeof(double));
  for (int64_t p = 0; p < nnz; p++) {
    int64_t s = slot[cidx[mode][p]];
    if (s < 0) continue;
    double* m = Mrows + s * R;
    double x = cvals[p];
    for (int r = 0; r < R; r++) {
      double w = 1.0;
      int first = 1;
      for (int k = 0; k < N; k++) {
        if (k == mode) continue;
        double hv = H[k][(int64_t)cidx[k][p] * R + r];
        w = first ? hv : w * hv;
        first = 0;
      }
      m[r] = m[r] + x * w;
    }
  }
  /* duplicated sample rows: copy from the slot that owns the row */
  for (int64_t s = 0; s < nrows; s++) {
    int64_t o = slot[rows[s]];
    if (o != s) memcpy(Mrows + s * R, Mrows + o * R, (size_t)R * sizeof(double));
  }
  free(slot);
  return ORC_OK;
}

/* ---------------- O3: Gram G = H^T H (Alg. 1 l.4, l.12) ------------------------------ */
int oracle_gram(int64_t I, int R, const double* H, double* G) {
  int64_t nb = (I + BLK - 1) / BLK;
  double* part = (double*)calloc((size_t)((nb > 0 ? nb : 1) * R * R), sizeof(double));
  if (!part) return ORC_ENOMEM;
#pragma omp parallel for schedule(static)
  for (int64_t b = 0; b < nb; b++) {
    double* P = part + b * R * R;
    int64_t i1 = (b + 1) * BLK < I ? (b + 1) * BLK : I;
    for (int64_t i = b * BLK; i < i1; i++)
      for (int a = 0; a < R; a++)
        for (int c = 0; c < R; c++)
          P[a * R + c] = P[a * R + c] + H[i * R + a] * H[i * R + c];
  }
  for (int e = 0; e < R * R; e++) G[e] = 0.0;
  for (int64_t b = 0; b < nb; b++)
    for (int e = 0; e < R * R; e++) G[e] = G[e] + part[b * R * R + e];
  free(part);
  return ORC_OK;
}

/* ---------------- O4: S = *_{k != n} G^(k) (Alg. 1 l.8, L494) ------------------------ */
int oracle_hadamard_except(int N, int R, const double* const* G, int n, double* S) {
  int first = 1;
  for (int k = 0; k < N; k++) {
    if (k == n) continue;
    for (int e = 0; e < R * R; e++) S[e] = first ? G[k][e] : S[e] * G[k][e];
    first = 0;
  }
  if (first) for (int e = 0; e < R * R; e++) S[e] = 1.0;
  return ORC_OK;
}

/* ---------------- O6: Cholesky-Banachiewicz, A = L L^T (Alg. 2 l.3, L560) ----------- */
int oracle_cholesky(int R, const double* A, double* L) {
  for (int e = 0; e < R * R; e++) L[e] = 0.0;
  for (int i = 0; i < R; i++) {
    for (int j = 0; j <= i; j++) {
      double s = A[i * R + j];
      for (int k = 0; k < j; k++) s = s - L[i * R + k] * L[j * R + k];
      if (i == j) {
        if (!(s > 0.0)) return ORC_NOT_SPD;
        L[i * R + i] = sqrt(s);
      } else {
        L[i * R + j] = s / L[j * R + j];
      }
    }
  }
  return ORC_OK;
}

/* ---------------- O7: ADMM, Alg. 2 (L550-580) -----------------------------------------
 * rho = tr(S)/R unless rho_in > 0 (Alg. 2 l.2); L = chol(S + rho I) (l.3).
 * repeat (j = 1..max_iter):
 *   H0 <- H                                   (l.5, reading D2)
 *   H~ <- (L L^T)^{-1} (M + rho (H + U))      (l.6, row-major reading D1:
 *                                              forward then back substitution per row)
 *   H  <- prox(H~ - U)                        (l.7; nonneg: x > 0 ? x : +0.0, D15;
 *                                              L1 variants threshold at alpha/rho,
 *                                              the box clips to [0, alpha])
 *   U  <- U + H - H~                          (l.8)
 * until ||H - H~||^2 < eps ||H||^2 and ||H - H0||^2 < eps ||U||^2 (l.9, reading D3:
 *   squared norms of the UPDATED H, U, strict <, no division, at least one pass).
 * stats = {iters, rho, r, s, nH, nU} of the last pass; trace (optional) gets the
 * four sums of every pass [max_iter][4]. */
int oracle_admm(int64_t I, int R, const double* M, const double* S, double* H, double* U,
                double tol, int max_iter, double rho_in, int prox, double alpha, double* stats, double* trace) {
  if (R < 1 || max_iter < 1 || I < 0) return ORC_EINVAL;
  double rho = 0.0;
  if (rho_in > 0.0) rho = rho_in;
  else {
    double tr = 0.0;
    for (int a = 0; a < R; a++) tr = tr + S[a * R + a];
    rho = tr / R;
  }
  if (!(rho > 0.0)) return ORC_NOT_SPD;
  const double tau = alpha / rho;
  double* A = (double*)malloc((size_t)R * R * sizeof(double));
  double* L = (double*)malloc((size_t)R * R * sizeof(double));
  for (int e = 0; e < R * R; e++) A[e] = S[e];
  for (int a = 0; a < R; a++) A[a * R + a] = A[a * R + a] + rho;
  int st = oracle_cholesky(R, A, L);
  free(A);
  if (st) { free(L); return st; }
  int64_t nb = (I + BLK - 1) / BLK;
  double* part = (double*)malloc((size_t)((nb > 0 ? nb : 1) * 4) * sizeof(double));
  double r = 0, s = 0, nH = 0, nU = 0;
  int it = 0;
  for (int j = 1; j <= max_iter; j++) {
#pragma omp parallel for schedule(static)
    for (int64_t b = 0; b < nb; b++) {
      double t[128], y[128], x[128], h0[128];
      double pr = 0, ps = 0, ph = 0, pu = 0;
      int64_t i1 = (b + 1) * BLK < I ? (b + 1) * BLK : I;
      for (int64_t i = b * BLK; i < i1; i++) {
        const double* m = M + i * R;
        double* h = H + i * R;
        double* u = U + i * R;
        for (int c = 0; c < R; c++) { h0[c] = h[c]; t[c] = m[c] + rho * (h[c] + u[c]); }
        for (int a = 0; a < R; a++) {              /* L y = t */
          double v = t[a];
          for (int k = 0; k < a; k++) v = v - L[a * R + k] * y[k];
          y[a] = v / L[a * R + a];
        }
        for (int a = R - 1; a >= 0; a--) {         /* L^T x = y */
          double v = y[a];
          for (int k = a + 1; k < R; k++) v = v - L[k * R + a] * x[k];
          x[a] = v / L[a * R + a];
        }
        for (int c = 0; c < R; c++) {
          double d = x[c] - u[c];
          double hn = prox_apply(prox, d, tau, alpha);
          double un = u[c] + hn - x[c];
          double e1 = hn - x[c], e2 = hn - h0[c];
          pr = pr + e1 * e1; ps = ps + e2 * e2; ph = ph + hn * hn; pu = pu + un * un;
          h[c] = hn; u[c] = un;
        }
      }
      part[b * 4 + 0] = pr; part[b * 4 + 1] = ps; part[b * 4 + 2] = ph; part[b * 4 + 3] = pu;
    }
    r = s = nH = nU = 0.0;
    for (int64_t b = 0; b < nb; b++) {
      r = r + part[b * 4 + 0]; s = s + part[b * 4 + 1];
      nH = nH + part[b * 4 + 2]; nU = nU + part[b * 4 + 3];
    }
    if (trace) { trace[(j - 1) * 4 + 0] = r; trace[(j - 1) * 4 + 1] = s; trace[(j - 1) * 4 + 2] = nH; trace[(j - 1) * 4 + 3] = nU; }
    it = j;
    if (!isfinite(r) || !isfinite(s) || !isfinite(nH) || !isfinite(nU)) { free(L); free(part); return ORC_NUMERIC; }
    if (r < tol * nH && s < tol * nU) break;
  }
  if (stats) { stats[0] = it; stats[1] = rho; stats[2] = r; stats[3] = s; stats[4] = nH; stats[5] = nU; }
  free(L); free(part);
  return ORC_OK;
}

/* ---------------- f1: HALS and MU updates (Sec. 5.4) ---------------------
 * The paper plugs two more non-negativity schemes into the same framework
 * (AUNTF_GPU, L717-722) without spelling them out; readings D21 / D22:
 *  HALS [4], one sweep per row, columns in order (Gauss-Seidel inside the row):
 *     h_r <- max(0, h_r + (m_r - sum_k h_k S[k][r]) / S[r][r])   (S[r][r] > 0; else h_r kept)
 *  MU [14], all columns at once from the previous h:
 *     h_r <- h_r * m_r / (sum_k h_k S[k][r] + 1e-16)
 * `sweeps` passes over every row. */
#define MU_EPS 1e-16
int oracle_hals(int64_t I, int R, const double* M, const double* S, double* H, int sweeps) {
  if (R < 1 || R > 128 || sweeps < 1) return ORC_EINVAL;
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < I; i++) {
    const double* m = M + i * R;
    double* h = H + i * R;
    for (int sw = 0; sw < sweeps; sw++)
      for (int r = 0; r < R; r++) {
        const double d = S[r * R + r];
        if (!(d > 0.0)) continue;
        double dot = 0.0;
        for (int k = 0; k < R; k++) dot = dot + h[k] * S[k * R + r];
        const double v = h[r] + (m[r] - dot) / d;
        h[r] = v > 0.0 ? v : 0.0;
      }
  }
  return ORC_OK;
}

int oracle_mu(int64_t I, int R, const double* M, const double* S, double* H, int sweeps) {
  if (R < 1 || R > 128 || sweeps < 1) return ORC_EINVAL;
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < I; i++) {
    const double* m = M + i * R;
    double* h = H + i * R;
    double den[128];
    for (int sw = 0; sw < sweeps; sw++) {
      for (int r = 0; r < R; r++) {
        double dot = 0.0;
        for (int k = 0; k < R; k++) dot = dot + h[k] * S[k * R + r];
        den[r] = dot + MU_EPS;
      }
      for (int r = 0; r < R; r++) h[r] = h[r] * m[r] / den[r];
    }
  }
  return ORC_OK;
}

/* ---------------- O8: normalize (Alg. 1 l.11, L499; readings D7, D8) ------------------
 * lambda_r = sqrt(sum_i h_ir^2); if lambda_r > 0 the column is divided by it. */
int oracle_normalize(int64_t I, int R, double* H, double* lam) {
  int64_t nb = (I + BLK - 1) / BLK;
  double* part = (double*)calloc((size_t)((nb > 0 ? nb : 1) * R), sizeof(double));
  if (!part) return ORC_ENOMEM;
#pragma omp parallel for schedule(static)
  for (int64_t b = 0; b < nb; b++) {
    int64_t i1 = (b + 1) * BLK < I ? (b + 1) * BLK : I;
    for (int64_t i = b * BLK; i < i1; i++)
      for (int c = 0; c < R; c++) part[b * R + c] = part[b * R + c] + H[i * R + c] * H[i * R + c];
  }
  for (int c = 0; c < R; c++) {
    double s = 0.0;
    for (int64_t b = 0; b < nb; b++) s = s + part[b * R + c];
    lam[c] = sqrt(s);
  }
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < I; i++)
    for (int c = 0; c < R; c++)
      if (lam[c] > 0.0) H[i * R + c] = H[i * R + c] / lam[c];
  free(part);
  return ORC_OK;
}

/* ---------------- O10: fit (reading D12) ----------------------------------------------
 * fit = 1 - sqrt(max(0, ||X||^2 + lam^T (*_k G^(k)) lam - 2 sum_{i,r} M_ir H_ir lam_r)) / ||X||
 * with M = MTTKRP of the last mode, H its normalised factor, lam its norms. */
double oracle_fit(int N, int R, double normX2, int64_t I_last, const double* M_last,
                  const double* H_last, const double* lam, const double* const* G) {
  double xhat = 0.0;
  for (int a = 0; a < R; a++)
    for (int b = 0; b < R; b++) {
      double g = 1.0;
      for (int k = 0; k < N; k++) g = g * G[k][a * R + b];
      xhat = xhat + lam[a] * lam[b] * g;
    }
  int64_t nb = (I_last + BLK - 1) / BLK;
  double* part = (double*)calloc((size_t)(nb > 0 ? nb : 1), sizeof(double));
#pragma omp parallel for schedule(static)
  for (int64_t b = 0; b < nb; b++) {
    int64_t i1 = (b + 1) * BLK < I_last ? (b + 1) * BLK : I_last;
    double p = 0.0;
    for (int64_t i = b * BLK; i < i1; i++)
      for (int c = 0; c < R; c++) p = p + M_last[i * R + c] * H_last[i * R + c] * lam[c];
    part[b] = p;
  }
  double inner = 0.0;
  for (int64_t b = 0; b < nb; b++) inner = inner + part[b];
  free(part);
  double res2 = normX2 + xhat - 2.0 * inner;
  if (res2 < 0.0) res2 = 0.0;
  return 1.0 - sqrt(res2) / sqrt(normX2);
}

/* ---------------- O9/O11: Alg. 1 outer loop ---------------------------------------------
 * State per mode n: H^(n) (normalised, in/out), lambda^(n), dual U^(n) (zero at
 * start, persists across outer iterations: reading D4), G^(n) = H^(n)T H^(n).
 * normalize_init: column-normalise the caller's factors, lambda = 1 (reading D6).
 * for t = 1..outer_iters, for n = 1..N (Gauss-Seidel, D13):
 *   S = *_{k!=n} G^(k); M = MTTKRP(n);
 *   H = H^(n) diag(lambda^(n)) (warm = 0, scaled, D4) or H^(n) (warm = 1, literal Alg. 1);
 *   ADMM(S, M, H, U^(n)); (H^(n), lambda^(n)) = normalize(H); G^(n) = H^(n)T H^(n)
 * then fit; stop early if fit_tol > 0 and |fit - fit_prev| < fit_tol (D11).
 * update: 0 ADMM (Alg. 2), 1 HALS, 2 MU (f1; max_iter sweeps, S unused by rho).
 * lam_all: N*R output (every mode's lambda; the Kruskal lambda is the last mode's, D10).
 * phase_ms[4] += GRAM, MTTKRP, UPDATE, NORMALIZE wall times.
 * trace_out (optional) [outer_iters][N][max_iter][4]: the four sums of every ADMM
 * pass (r, s, nH, nU), used by tests to measure the stop-test margin (U2). */
int oracle_factorize(int N, const int64_t* dims, int64_t nnz, const int32_t* const* cidx,
                     const double* cvals, double normX2, int R, int outer_iters, double fit_tol,
                     double tol, int max_iter, double rho_in, int warm, int normalize_init, int prox,
                     double alpha, int update, double* const* H, double* lam_all, double* fit_out, int* iters_out,
                     int* outer_done, double* phase_ms, double* trace_out) {
  if (N < 2 || N > 8 || R < 1 || R > 128 || outer_iters < 1 || max_iter < 1) return ORC_EINVAL;
  int st = ORC_OK;
  double* G[8]; double* U[8];
  int64_t Imax = 0;
  for (int n = 0; n < N; n++) if (dims[n] > Imax) Imax = dims[n];
  double* M = (double*)malloc((size_t)(Imax * R) * sizeof(double));
  double* S = (double*)malloc((size_t)R * R * sizeof(double));
  for (int n = 0; n < N; n++) {
    G[n] = (double*)malloc((size_t)R * R * sizeof(double));
    U[n] = (double*)calloc((size_t)(dims[n] * R), sizeof(double));
    double* lam = lam_all + n * R;
    if (normalize_init) {
      oracle_normalize(dims[n], R, H[n], lam);
      for (int c = 0; c < R; c++) lam[c] = 1.0;
    } else {
      for (int c = 0; c < R; c++) lam[c] = 1.0;
    }
    oracle_gram(dims[n], R, H[n], G[n]);
  }
  double fit_prev = 0.0;
  int done = 0;
  for (int t = 0; t < outer_iters && st == ORC_OK; t++) {
    for (int n = 0; n < N; n++) {
      double t0 = now_ms();
      oracle_hadamard_except(N, R, (const double* const*)G, n, S);
      double t1 = now_ms();
      st = oracle_mttkrp(N, dims, nnz, cidx, cvals, n, R, (const double* const*)H, M);
      if (st) break;
      double t2 = now_ms();
      double* lam = lam_all + n * R;
      if (warm == 0) {
        for (int64_t i = 0; i < dims[n]; i++)
          for (int c = 0; c < R; c++) H[n][i * R + c] = H[n][i * R + c] * lam[c];
      }
      double stats[6];
      double* tr = trace_out ? trace_out + ((size_t)t * N + n) * (size_t)max_iter * 4 : NULL;
      if (update == 1) st = oracle_hals(dims[n], R, M, S, H[n], max_iter);
      else if (update == 2) st = oracle_mu(dims[n], R, M, S, H[n], max_iter);
      else st = oracle_admm(dims[n], R, M, S, H[n], U[n], tol, max_iter, rho_in, prox, alpha, stats, tr);
      if (st) break;
      if (iters_out) iters_out[t * N + n] = update ? max_iter : (int)stats[0];
      double t3 = now_ms();
      oracle_normalize(dims[n], R, H[n], lam);
      double t4 = now_ms();
      oracle_gram(dims[n], R, H[n], G[n]);
      double t5 = now_ms();
      if (phase_ms) {
        phase_ms[0] += (t1 - t0) + (t5 - t4);
        phase_ms[1] += t2 - t1;
        phase_ms[2] += t3 - t2;
        phase_ms[3] += t4 - t3;
      }
    }
    if (st) break;
    double fit = oracle_fit(N, R, normX2, dims[N - 1], M, H[N - 1], lam_all + (N - 1) * R,
                            (const double* const*)G);
    if (!isfinite(fit)) { st = ORC_NUMERIC; break; }
    if (fit_out) fit_out[t] = fit;
    done = t + 1;
    if (fit_tol > 0.0 && t > 0 && fabs(fit - fit_prev) < fit_tol) break;
    fit_prev = fit;
  }
  if (outer_done) *outer_done = done;
  for (int n = 0; n < N; n++) { free(G[n]); free(U[n]); }
  free(M); free(S);
  return st;
}
