// Sparse MTTKRP (hot-path step a2): PAPER.md Fig. 2 (L403-430), Alg. 1 l.9.
//   M[i, :] = sum_{nonzeros x with i_mode = i} x * (*_{k != mode} H^(k)[i_k, :])
//
// B200 design: the mode-n copy of the store is sorted by
// i_n with an int64 row pointer.  Work is split into equal nonzero chunks (one
// warp each, lanes = factor columns) so heavy rows of power-law modes are
// shared by many warps.  A chunk owns the rows whose first nonzero lies in it
// and writes them directly (coalesced, no atomics); the head of a row that
// started in an earlier chunk goes to a per-chunk carry slot, added by a
// fix-up pass in chunk order.  Fixed chunking + fixed order => deterministic,
// no floating-point atomics.  Factor rows (R*8 bytes) are gathered whole by
// one warp-wide load; nonzero metadata is loaded 32 at a time and broadcast
// with shuffles.
#include "internal.h"

namespace cstf {
namespace {

constexpr int kWarps = 8;  // per CTA

struct MArgs {
  const int64_t* rowptr;
  const int32_t* idx[7];
  const double* F[7];
  const double* vals;
  int64_t I, nnz, chunk, nchunks;
  int R;
  const int64_t* lb;    // [nchunks+1] first row with rowptr >= c*chunk (lb[nchunks] = I)
  const int32_t* cont;  // [nchunks] row continuing into chunk c from an earlier chunk, or -1
  double* M;
  double* carry;        // [nchunks][R]
};

__global__ void k_chunk_bounds(const int64_t* __restrict__ rowptr, int64_t I, int64_t nnz,
                               int64_t chunk, int64_t nchunks, int64_t* __restrict__ lb,
                               int32_t* __restrict__ cont) {
  for (int64_t c = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; c <= nchunks;
       c += (int64_t)gridDim.x * blockDim.x) {
    if (c == nchunks) { lb[c] = I; continue; }
    int64_t p0 = c * chunk;
    // lower_bound: first row r with rowptr[r] >= p0
    int64_t lo = 0, hi = I;
    while (lo < hi) {
      int64_t mid = (lo + hi) >> 1;
      if (rowptr[mid] < p0) lo = mid + 1; else hi = mid;
    }
    lb[c] = lo;
    // row containing p0 started before p0?  it is lo-1 when rowptr[lo] > p0 or lo == I
    int32_t ct = -1;
    if (p0 < nnz && lo > 0 && (lo == I || rowptr[lo] > p0)) ct = (int32_t)(lo - 1);
    cont[c] = ct;
  }
}

template <int NOTHER, int CPL, bool VEC>
__global__ void __launch_bounds__(kWarps * 32) k_mttkrp(MArgs a) {
  const int lane = threadIdx.x & 31;
  const int64_t warp0 = blockIdx.x * (int64_t)kWarps + (threadIdx.x >> 5);
  const int64_t nwarps = (int64_t)gridDim.x * kWarps;
  const int R = a.R;
  int col[CPL];
  bool cok[CPL];
#pragma unroll
  for (int s = 0; s < CPL; s++) {
    col[s] = VEC ? lane * CPL + s : lane + 32 * s;
    cok[s] = col[s] < R;
  }
  for (int64_t c = warp0; c < a.nchunks; c += nwarps) {
    const int64_t p0 = c * a.chunk;
    const int64_t p1 = min(p0 + a.chunk, a.nnz);
    const int32_t ct = a.cont[c];
    int64_t row = ct >= 0 ? (int64_t)ct : a.lb[c];
    const int64_t row_end = (c == a.nchunks - 1) ? a.I : a.lb[c + 1];
    double acc[CPL];
#pragma unroll
    for (int s = 0; s < CPL; s++) acc[s] = 0.0;
    int64_t seg_end = (row < row_end) ? min(a.rowptr[row + 1], p1) : p1;

    auto flush = [&](int64_t r) {
      double* dst = (ct >= 0 && r == (int64_t)ct) ? a.carry + c * (int64_t)R : a.M + r * (int64_t)R;
      if (VEC) {
        if (CPL == 2) {
          if (cok[0]) reinterpret_cast<double2*>(dst)[lane] = make_double2(acc[0], acc[1]);
        } else {
#pragma unroll
          for (int s = 0; s < CPL; s += 2)
            if (cok[s]) reinterpret_cast<double2*>(dst + col[s])[0] = make_double2(acc[s], acc[s + 1]);
        }
      } else {
#pragma unroll
        for (int s = 0; s < CPL; s++)
          if (cok[s]) dst[col[s]] = acc[s];
      }
#pragma unroll
      for (int s = 0; s < CPL; s++) acc[s] = 0.0;
    };

    for (int64_t pb = p0; pb < p1; pb += 32) {
      const int nb = (int)min((int64_t)32, p1 - pb);
      int jreg[NOTHER];
      double vreg = 0.0;
      if (lane < nb) {
#pragma unroll
        for (int q = 0; q < NOTHER; q++) jreg[q] = __ldg(a.idx[q] + pb + lane);
        vreg = __ldg(a.vals + pb + lane);
      } else {
#pragma unroll
        for (int q = 0; q < NOTHER; q++) jreg[q] = 0;
      }
      int t = 0;
      while (t < nb) {
        const int64_t p = pb + t;
        if (p >= seg_end) {
          flush(row);
          row++;
          seg_end = min(a.rowptr[row + 1], p1);
          continue;
        }
        int run = (int)min((int64_t)(nb - t), seg_end - p);
        // unrolled by 4 for memory-level parallelism
        for (; run >= 4; run -= 4, t += 4) {
          double v[4];
          double w[4][CPL];
#pragma unroll
          for (int u = 0; u < 4; u++) {
            v[u] = __shfl_sync(0xffffffffu, vreg, t + u);
#pragma unroll
            for (int q = 0; q < NOTHER; q++) {
              const int j = __shfl_sync(0xffffffffu, jreg[q], t + u);
              const double* src = a.F[q] + (int64_t)j * R;
              double f[CPL];
              if (VEC) {
#pragma unroll
                for (int s = 0; s < CPL; s += 2) {
                  double2 x = cok[s] ? __ldg(reinterpret_cast<const double2*>(src + col[s])) : make_double2(0.0, 0.0);
                  f[s] = x.x; f[s + 1] = x.y;
                }
              } else {
#pragma unroll
                for (int s = 0; s < CPL; s++) f[s] = cok[s] ? __ldg(src + col[s]) : 0.0;
              }
#pragma unroll
              for (int s = 0; s < CPL; s++) w[u][s] = (q == 0) ? f[s] : w[u][s] * f[s];
            }
          }
#pragma unroll
          for (int u = 0; u < 4; u++)
#pragma unroll
            for (int s = 0; s < CPL; s++) acc[s] = fma(v[u], w[u][s], acc[s]);
        }
        for (; run > 0; run--, t++) {
          const double v = __shfl_sync(0xffffffffu, vreg, t);
          double w[CPL];
#pragma unroll
          for (int q = 0; q < NOTHER; q++) {
            const int j = __shfl_sync(0xffffffffu, jreg[q], t);
            const double* src = a.F[q] + (int64_t)j * R;
            double f[CPL];
            if (VEC) {
#pragma unroll
              for (int s = 0; s < CPL; s += 2) {
                double2 x = cok[s] ? __ldg(reinterpret_cast<const double2*>(src + col[s])) : make_double2(0.0, 0.0);
                f[s] = x.x; f[s + 1] = x.y;
              }
            } else {
#pragma unroll
              for (int s = 0; s < CPL; s++) f[s] = cok[s] ? __ldg(src + col[s]) : 0.0;
            }
#pragma unroll
            for (int s = 0; s < CPL; s++) w[s] = (q == 0) ? f[s] : w[s] * f[s];
          }
#pragma unroll
          for (int s = 0; s < CPL; s++) acc[s] = fma(v, w[s], acc[s]);
        }
      }
    }
    // the row in progress, then owned empty rows up to row_end
    while (row < row_end) {
      flush(row);
      row++;
    }
  }
}

// Add the carries of every row that continues across chunks, in chunk order.
__global__ void k_carry_fixup(const int32_t* __restrict__ cont, int64_t nchunks,
                              const double* __restrict__ carry, int R, double* __restrict__ M) {
  const int lane = threadIdx.x & 31;
  const int64_t warp0 = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t c = warp0; c < nchunks; c += nwarps) {
    const int32_t h = cont[c];
    if (h < 0 || (c > 0 && cont[c - 1] == h)) continue;
    for (int col = lane; col < R; col += 32) {
      double s = 0.0;
      for (int64_t cc = c; cc < nchunks && cont[cc] == h; cc++) s += carry[cc * R + col];
      M[(int64_t)h * R + col] += s;
    }
  }
}

template <int NOTHER>
cstf_status launch_main(const MArgs& a, int grid, cudaStream_t st) {
  const int R = a.R;
  if (R == 64) {
    k_mttkrp<NOTHER, 2, true><<<grid, kWarps * 32, 0, st>>>(a);
  } else if (R == 128) {
    k_mttkrp<NOTHER, 4, true><<<grid, kWarps * 32, 0, st>>>(a);
  } else if (R <= 32) {
    k_mttkrp<NOTHER, 1, false><<<grid, kWarps * 32, 0, st>>>(a);
  } else if (R <= 64) {
    k_mttkrp<NOTHER, 2, false><<<grid, kWarps * 32, 0, st>>>(a);
  } else {
    k_mttkrp<NOTHER, 4, false><<<grid, kWarps * 32, 0, st>>>(a);
  }
  CSTF_LAUNCHED();
  return CSTF_OK;
}

struct Workspace {
  DevBuf lb, cont, carry;
};
Workspace& ws() {
  static thread_local Workspace w[64];
  int dev = 0;
  cudaGetDevice(&dev);
  return w[dev & 63];
}

}  // namespace

cstf_status mttkrp(const cstf_tensor* X, int mode, int R, const double* const* d_factors,
                   double* d_M, cudaStream_t st, int64_t* launches) {
  const ModeStore& ms = X->mode[mode];
  const int N = X->N;
  const DeviceInfo& di = device_info();
  const int64_t nnz = ms.nnz;
  // chunk: ~4 chunks per resident warp, multiple of 32, in [256, 8192]
  const int64_t resident = (int64_t)di.sms * 8 * kWarps;
  int64_t chunk = (nnz + resident * 4 - 1) / (resident * 4);
  chunk = ((chunk + 31) / 32) * 32;
  if (chunk < 256) chunk = 256;
  if (chunk > 8192) chunk = 8192;
  const int64_t nchunks = nnz > 0 ? (nnz + chunk - 1) / chunk : 1;
  Workspace& w = ws();
  CSTF_TRY(w.lb.ensure((size_t)(nchunks + 1) * 8));
  CSTF_TRY(w.cont.ensure((size_t)nchunks * 4));
  CSTF_TRY(w.carry.ensure((size_t)nchunks * R * 8));
  MArgs a;
  a.rowptr = ms.rowptr.as<int64_t>();
  for (int q = 0; q < N - 1; q++) {
    a.idx[q] = ms.idx[q].as<int32_t>();
    a.F[q] = d_factors[ms.other[q]];
  }
  a.vals = ms.vals.as<double>();
  a.I = ms.I;
  a.nnz = nnz;
  a.chunk = chunk;
  a.nchunks = nchunks;
  a.R = R;
  a.lb = w.lb.as<int64_t>();
  a.cont = w.cont.as<int32_t>();
  a.M = d_M;
  a.carry = w.carry.as<double>();
  if (ms.I == 0) return CSTF_OK;
  {
    int g = (int)std::min<int64_t>((nchunks + 1 + 255) / 256, (int64_t)di.sms * 8);
    k_chunk_bounds<<<g, 256, 0, st>>>(a.rowptr, ms.I, nnz, chunk, nchunks, w.lb.as<int64_t>(),
                                       w.cont.as<int32_t>());
    CSTF_LAUNCHED();
  }
  const int grid = (int)std::min<int64_t>((nchunks + kWarps - 1) / kWarps, (int64_t)di.sms * 8);
  switch (N - 1) {
    case 1: CSTF_TRY(launch_main<1>(a, grid, st)); break;
    case 2: CSTF_TRY(launch_main<2>(a, grid, st)); break;
    case 3: CSTF_TRY(launch_main<3>(a, grid, st)); break;
    case 4: CSTF_TRY(launch_main<4>(a, grid, st)); break;
    case 5: CSTF_TRY(launch_main<5>(a, grid, st)); break;
    case 6: CSTF_TRY(launch_main<6>(a, grid, st)); break;
    case 7: CSTF_TRY(launch_main<7>(a, grid, st)); break;
    default: return fail(CSTF_ERR_UNSUPPORTED, "nmodes");
  }
  if (nchunks > 1) {
    int g = (int)std::min<int64_t>((nchunks * 32 + 255) / 256, (int64_t)di.sms * 8);
    k_carry_fixup<<<g, 256, 0, st>>>(a.cont, nchunks, a.carry, R, d_M);
    CSTF_LAUNCHED();
  }
  if (launches) *launches += (nchunks > 1) ? 3 : 2;
  return CSTF_OK;
}

}  // namespace cstf
