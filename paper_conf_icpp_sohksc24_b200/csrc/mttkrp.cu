// Sparse MTTKRP (hot-path step a2): PAPER.md Fig. 2 (L403-430), Alg. 1 l.9.
//   M[i, :] = sum_{nonzeros x with i_mode = i} x * (*_{k != mode} H^(k)[i_k, :])
//
// B200 design:
//  * The mode-n copy of the store is sorted by i_n and, inside a row, by the
//    other modes in increasing length; each nonzero is one 16/32-byte record
//    {indices..., x}; a warp reads 32 records with coalesced 16-byte loads.
//  * Work is split into equal nonzero chunks, one warp each, so the heavy rows
//    of power-law modes are shared by many warps.  A chunk owns the rows whose
//    first nonzero lies in it and writes them directly (coalesced, no atomics);
//    the head of a row that started earlier goes to a per-chunk carry slot,
//    added by a fix-up pass in chunk order.  Fixed chunking + fixed order =>
//    deterministic, no floating-point atomics.
//  * A group of G = min(32, R/2) lanes covers one factor row with 16-byte
//    loads; the P = 32/G groups of a warp take interleaved nonzeros of the
//    same row and are combined with xor-shuffles when the row is written.
//    Consecutive nonzeros of a fiber (same index of the shortest other mode)
//    are gathered back to back, so the repeated fiber row is an L1 hit.
//  * Measured bound: with L2-resident factors the kernel runs at
//    the L2->SM row-gather rate (~20 TB/s on B200 for 256-byte rows).
#include "internal.h"

namespace cstf {
namespace {

constexpr int kWarps = 8;  // per CTA

struct MArgs {
  const int64_t* rowptr;
  const char* rec;
  const double* F[7];   // factor of record slot q
  int64_t I, nnz, chunk, nchunks;
  int R, recb, nother;
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
    const int64_t p0 = c * chunk;
    int64_t lo = 0, hi = I;          // lower_bound: first row r with rowptr[r] >= p0
    while (lo < hi) {
      const int64_t mid = (lo + hi) >> 1;
      if (rowptr[mid] < p0) lo = mid + 1; else hi = mid;
    }
    lb[c] = lo;
    int32_t ct = -1;                 // the row containing p0 started before p0
    if (p0 < nnz && lo > 0 && (lo == I || rowptr[lo] > p0)) ct = (int32_t)(lo - 1);
    cont[c] = ct;
  }
}

// base + j * ROWB as one wide multiply-add
template <unsigned ROWB>
__device__ __forceinline__ const double2* row_addr(const char* base, unsigned j) {
  const double2* p;
  asm("mad.wide.u32 %0, %1, %2, %3;" : "=l"(p) : "r"(j), "n"(ROWB), "l"(base));
  return p;
}

// Fast path: R in {2, 4, 8, 16, 32, 64, 128}, records of 16 or 32 bytes.
// The warp loads 32 records at a time (one coalesced 16-byte load per lane and
// record word group) and broadcasts them with shuffles; the P groups take
// interleaved nonzeros of the current row, so consecutive nonzeros of a fiber
// are gathered back to back and the repeated fiber row hits in L1.
template <int NOTHER, int R, int RECB>
__global__ void __launch_bounds__(kWarps * 32, 2) k_mttkrp_fast(MArgs a) {
  constexpr int RV = R / 2;                    // double2 per row
  constexpr int G = RV < 32 ? RV : 32;         // lanes per group
  constexpr int VPL = RV / G;                  // double2 per lane
  constexpr int P = 32 / G;                    // nonzeros per warp step
  constexpr unsigned ROWB = R * 8;
  constexpr int NW = RECB / 4;                 // 32-bit words per record
  const int lane = threadIdx.x & 31;
  const int sg = lane / G, gl = lane % G;
  const int64_t warp0 = blockIdx.x * (int64_t)kWarps + (threadIdx.x >> 5);
  const int64_t nwarps = (int64_t)gridDim.x * kWarps;
  const char* Fb[NOTHER];
#pragma unroll
  for (int q = 0; q < NOTHER; q++) Fb[q] = reinterpret_cast<const char*>(a.F[q]) + gl * 16;
  for (int64_t c = warp0; c < a.nchunks; c += nwarps) {
    const int64_t p0 = c * a.chunk;
    const int64_t p1 = min(p0 + a.chunk, a.nnz);
    const int32_t ct = a.cont[c];
    int64_t row = ct >= 0 ? (int64_t)ct : a.lb[c];
    const int64_t row_end = (c == a.nchunks - 1) ? a.I : a.lb[c + 1];
    double2 acc[VPL];
#pragma unroll
    for (int s = 0; s < VPL; s++) acc[s] = make_double2(0.0, 0.0);
    int64_t seg_end = (row < row_end) ? min(a.rowptr[row + 1], p1) : p1;

    auto flush = [&](int64_t r) {
#pragma unroll
      for (int off = 16; off >= G; off >>= 1)
#pragma unroll
        for (int s = 0; s < VPL; s++) {
          acc[s].x += __shfl_xor_sync(0xffffffffu, acc[s].x, off);
          acc[s].y += __shfl_xor_sync(0xffffffffu, acc[s].y, off);
        }
      if (sg == 0) {
        double* dst = (ct >= 0 && r == (int64_t)ct) ? a.carry + c * (int64_t)R : a.M + r * (int64_t)R;
#pragma unroll
        for (int s = 0; s < VPL; s++) reinterpret_cast<double2*>(dst)[gl + s * G] = acc[s];
      }
#pragma unroll
      for (int s = 0; s < VPL; s++) acc[s] = make_double2(0.0, 0.0);
    };

    for (int64_t pb = p0; pb < p1; pb += 32) {
      const int nb = (int)min((int64_t)32, p1 - pb);
      unsigned w[NW];
      if (lane < nb) {
        const int4* rp = reinterpret_cast<const int4*>(a.rec + (pb + lane) * RECB);
#pragma unroll
        for (int k = 0; k < NW / 4; k++) {
          const int4 x = __ldcs(rp + k);
          w[4 * k] = x.x; w[4 * k + 1] = x.y; w[4 * k + 2] = x.z; w[4 * k + 3] = x.w;
        }
      } else {
#pragma unroll
        for (int k = 0; k < NW; k++) w[k] = 0u;
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
        const int run = (int)min((int64_t)(nb - t), seg_end - p);
        for (int done = 0; done < run; done += P) {
          const bool ok = (done + sg) < run;
          const int srcc = ok ? t + done + sg : t + done;     // a valid lane of this batch
          const unsigned vlo = __shfl_sync(0xffffffffu, w[NW - 2], srcc);
          const unsigned vhi = __shfl_sync(0xffffffffu, w[NW - 1], srcc);
          const double v = ok ? __hiloint2double((int)vhi, (int)vlo) : 0.0;   // idle group adds 0
          double2 f[VPL];
#pragma unroll
          for (int q = 0; q < NOTHER; q++) {
            const unsigned j = __shfl_sync(0xffffffffu, w[q], srcc);
            const double2* rp = row_addr<ROWB>(Fb[q], j);
#pragma unroll
            for (int s = 0; s < VPL; s++) {
              const double2 x = __ldg(rp + s * G);
              if (q == 0) f[s] = x;
              else { f[s].x *= x.x; f[s].y *= x.y; }
            }
          }
#pragma unroll
          for (int s = 0; s < VPL; s++) {
            acc[s].x = fma(v, f[s].x, acc[s].x);
            acc[s].y = fma(v, f[s].y, acc[s].y);
          }
        }
        t += run;
      }
    }
    while (row < row_end) {
      flush(row);
      row++;
    }
  }
}

// Generic path (any R <= 128, any record size): lane = column(s), one nonzero at a time.
template <int CPL>
__global__ void __launch_bounds__(kWarps * 32) k_mttkrp_generic(MArgs a) {
  const int lane = threadIdx.x & 31;
  const int64_t warp0 = blockIdx.x * (int64_t)kWarps + (threadIdx.x >> 5);
  const int64_t nwarps = (int64_t)gridDim.x * kWarps;
  const int R = a.R;
  for (int64_t c = warp0; c < a.nchunks; c += nwarps) {
    const int64_t p0 = c * a.chunk;
    const int64_t p1 = min(p0 + a.chunk, a.nnz);
    const int32_t ct = a.cont[c];
    int64_t row = ct >= 0 ? (int64_t)ct : a.lb[c];
    const int64_t row_end = (c == a.nchunks - 1) ? a.I : a.lb[c + 1];
    int64_t seg0 = max(a.rowptr[row < row_end ? row : 0], p0);
    for (; row < row_end; row++) {
      const int64_t seg1 = min(a.rowptr[row + 1], p1);
      double acc[CPL];
#pragma unroll
      for (int s = 0; s < CPL; s++) acc[s] = 0.0;
      for (int64_t p = seg0; p < seg1; p++) {
        const char* r = a.rec + p * a.recb;
        const double v = *reinterpret_cast<const double*>(r + a.recb - 8);
        double w[CPL];
        for (int q = 0; q < a.nother; q++) {
          const unsigned j = reinterpret_cast<const unsigned*>(r)[q];
          const double* src = a.F[q] + (size_t)j * (unsigned)R;
#pragma unroll
          for (int s = 0; s < CPL; s++) {
            const int col = lane + 32 * s;
            const double f = col < R ? __ldg(src + col) : 0.0;
            w[s] = (q == 0) ? f : w[s] * f;
          }
        }
#pragma unroll
        for (int s = 0; s < CPL; s++) acc[s] = fma(v, w[s], acc[s]);
      }
      double* dst = (ct >= 0 && row == (int64_t)ct) ? a.carry + c * (int64_t)R : a.M + row * (int64_t)R;
#pragma unroll
      for (int s = 0; s < CPL; s++)
        if (lane + 32 * s < R) dst[lane + 32 * s] = acc[s];
      seg0 = seg1;
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

template <int NOTHER, int RECB>
bool launch_fast(const MArgs& a, int grid, cudaStream_t st) {
  switch (a.R) {
#define CASE(RR) case RR: k_mttkrp_fast<NOTHER, RR, RECB><<<grid, kWarps * 32, 0, st>>>(a); return true;
    CASE(2) CASE(4) CASE(8) CASE(16) CASE(32) CASE(64) CASE(128)
#undef CASE
    default: return false;
  }
}

cstf_status launch_main(const MArgs& a, int grid, cudaStream_t st) {
  bool done = false;
  switch (a.nother) {
    case 1: done = launch_fast<1, 16>(a, grid, st); break;
    case 2: done = launch_fast<2, 16>(a, grid, st); break;
    case 3: done = launch_fast<3, 32>(a, grid, st); break;
    case 4: done = launch_fast<4, 32>(a, grid, st); break;
    case 5: done = launch_fast<5, 32>(a, grid, st); break;
    case 6: done = launch_fast<6, 32>(a, grid, st); break;
    default: break;   // 7 other modes: 48-byte records, generic path
  }
  if (!done) {
    if (a.R <= 32) k_mttkrp_generic<1><<<grid, kWarps * 32, 0, st>>>(a);
    else if (a.R <= 64) k_mttkrp_generic<2><<<grid, kWarps * 32, 0, st>>>(a);
    else k_mttkrp_generic<4><<<grid, kWarps * 32, 0, st>>>(a);
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
  a.rec = ms.rec.as<char>();
  a.recb = ms.recb;
  a.nother = N - 1;
  for (int q = 0; q < N - 1; q++) a.F[q] = d_factors[ms.other[q]];
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
    const int g = (int)std::min<int64_t>((nchunks + 1 + 255) / 256, (int64_t)di.sms * 8);
    k_chunk_bounds<<<g, 256, 0, st>>>(a.rowptr, ms.I, nnz, chunk, nchunks, w.lb.as<int64_t>(),
                                       w.cont.as<int32_t>());
    CSTF_LAUNCHED();
  }
  const int grid = (int)std::min<int64_t>((nchunks + kWarps - 1) / kWarps, (int64_t)di.sms * 8);
  CSTF_TRY(launch_main(a, grid, st));
  if (nchunks > 1) {
    const int g = (int)std::min<int64_t>((nchunks * 32 + 255) / 256, (int64_t)di.sms * 8);
    k_carry_fixup<<<g, 256, 0, st>>>(a.cont, nchunks, a.carry, R, d_M);
    CSTF_LAUNCHED();
  }
  if (launches) *launches += (nchunks > 1) ? 3 : 2;
  return CSTF_OK;
}

}  // namespace cstf
