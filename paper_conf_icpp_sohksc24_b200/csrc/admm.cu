// ADMM update (hot-path step a5): cuADMM, Alg. 3 (L630-660) = Alg. 2
// (L550-580) with pre-inversion (Sec. 4.3.2) and operation fusion
// (Sec. 4.3.1).  Per row (reading D1, row-major):
//   H0 <- H;  H~ <- (M + rho (H + U)) Inv;  H <- prox(H~ - U);  U <- U + H - H~
//   r = ||H - H~||^2, s = ||H - H0||^2, nH = ||H||^2, nU = ||U||^2      (D3)
//
// B200 design:
//  * Rows are independent; only the four sums couple them.  A warp owns 8 rows
//    and keeps m, h, u in registers for ALL inner iterations of a launch
//    (row-resident, "v2"): HBM traffic is 5 I R words per launch instead of
//    per iteration.  One launch per iteration ("v1", streaming) uses the same
//    code with kiters = 1.
//  * The R x R product runs on the FP64 tensor-core path: mma.sync m8n8k4 f64
//    (SASS DMMA.8x8x4; tcgen05 has no f64 kind).  The accumulator (C) layout
//    of the product is reused as the A operand of the next iteration by
//    permuting the contraction index: thread (g = lane/4, q = lane%4) holds
//    row g, columns {8t + 2q, 8t + 2q + 1}; A chunk c of that thread is column
//    8(c/2) + 2q + (c%2), and the Inv fragment of chunk c is permuted the same
//    way, so no shuffles are needed between iterations.
//  * Per-iteration partial sums go to per-thread shared-memory slots and are
//    reduced in fixed order per CTA, then over CTAs by a finalize kernel that
//    also takes the stop decision on the device (deterministic).
#include "internal.h"

namespace cstf {
namespace {

constexpr int kThreads = 128;   // 4 warps
constexpr int kMaxK = 16;       // inner iterations per launch (chunk)

struct KArgs {
  const double* M;
  const double* H;
  const double* U;
  double* Hout;            // may alias H (in place) or be null (no write)
  double* Uout;
  const double* hscale;    // optional column scale of the incoming H
  int64_t I;
  int R;
  const double* inv;
  const double* scal;      // [0] = rho
  const int* flag;         // skip all work if a previous step failed
  int prox;
  int kiters;
  double* slots;           // [kiters][gridDim][4]
};

__device__ __forceinline__ void dmma(double& d0, double& d1, double a, double b) {
  asm("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
      : "+d"(d0), "+d"(d1)
      : "d"(a), "d"(b));
}

// RP = padded rank (multiple of 8, <= 64).  INV_REGS: Inv fragments in registers (RP <= 32).
template <int RP, bool INV_REGS>
__global__ void __launch_bounds__(kThreads) k_admm_dmma(KArgs a) {
  constexpr int NT = RP / 8;       // n-tiles of 8 columns
  constexpr int NC = 2 * NT;       // k-chunks of 4
  extern __shared__ double smem[];
  double* sacc = smem;                                   // [kiters][4][kThreads]
  double* sinv = smem + (size_t)kMaxK * 4 * kThreads;    // [NC][NT][32] fragments (if !INV_REGS)
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int g = lane >> 2, q = lane & 3;
  const int R = a.R;
  const bool skip = *a.flag != 0;   // an earlier step failed: write zero sums, touch nothing
  const double rho = a.scal[0];
  const int kiters = a.kiters;
  for (int x = tid; x < kiters * 4 * kThreads; x += kThreads) sacc[x] = 0.0;
  // B fragments: thread (g' = lane/4, q' = lane%4) holds Inv[kperm(c, q')][8t + g']
  double binv[INV_REGS ? NC : 1][INV_REGS ? NT : 1];
#pragma unroll
  for (int c = 0; c < NC; c++)
#pragma unroll
    for (int t = 0; t < NT; t++) {
      const int k = 8 * (c >> 1) + 2 * q + (c & 1);
      const int n = 8 * t + g;
      const double v = (k < R && n < R) ? a.inv[k * R + n] : 0.0;
      if (INV_REGS) binv[INV_REGS ? c : 0][INV_REGS ? t : 0] = v;
      else sinv[(c * NT + t) * 32 + lane] = v;
    }
  __syncthreads();
  double hs[NT][2];
#pragma unroll
  for (int t = 0; t < NT; t++)
#pragma unroll
    for (int i = 0; i < 2; i++) {
      const int col = 8 * t + 2 * q + i;
      hs[t][i] = (a.hscale && col < R) ? a.hscale[col] : 1.0;
    }
  const bool full = (R == RP);
  const int64_t ngroups = (a.I + 7) / 8;
  const int64_t gw0 = (int64_t)blockIdx.x * (kThreads / 32) + warp;
  const int64_t gws = (int64_t)gridDim.x * (kThreads / 32);
  for (int64_t grp = skip ? ngroups : gw0; grp < ngroups; grp += gws) {
    const int64_t row = grp * 8 + g;
    const bool rok = row < a.I;
    double m[NT][2], h[NT][2], u[NT][2];
    const size_t base = (size_t)row * R;
#pragma unroll
    for (int t = 0; t < NT; t++) {
      const int col = 8 * t + 2 * q;
      if (full) {
        double2 mv = make_double2(0.0, 0.0), hv = mv, uv = mv;
        if (rok) {
          mv = __ldcs(reinterpret_cast<const double2*>(a.M + base + col));
          hv = __ldcs(reinterpret_cast<const double2*>(a.H + base + col));
          uv = __ldcs(reinterpret_cast<const double2*>(a.U + base + col));
        }
        m[t][0] = mv.x; m[t][1] = mv.y; h[t][0] = hv.x; h[t][1] = hv.y; u[t][0] = uv.x; u[t][1] = uv.y;
      } else {
#pragma unroll
        for (int i = 0; i < 2; i++) {
          const bool ok = rok && (col + i) < R;
          m[t][i] = ok ? a.M[base + col + i] : 0.0;
          h[t][i] = ok ? a.H[base + col + i] : 0.0;
          u[t][i] = ok ? a.U[base + col + i] : 0.0;
        }
      }
#pragma unroll
      for (int i = 0; i < 2; i++) h[t][i] = h[t][i] * hs[t][i];
    }
    for (int j = 0; j < kiters; j++) {
      double d[NT][2];
#pragma unroll
      for (int t = 0; t < NT; t++) { d[t][0] = 0.0; d[t][1] = 0.0; }
#pragma unroll
      for (int c = 0; c < NC; c++) {
        const int tt = c >> 1, ii = c & 1;
        const double av = fma(rho, h[tt][ii] + u[tt][ii], m[tt][ii]);   // M + rho (H + U)
#pragma unroll
        for (int t = 0; t < NT; t++) {
          const double bv = INV_REGS ? binv[INV_REGS ? c : 0][INV_REGS ? t : 0] : sinv[(c * NT + t) * 32 + lane];
          dmma(d[t][0], d[t][1], av, bv);
        }
      }
      double pr = 0.0, ps = 0.0, ph = 0.0, pu = 0.0;
#pragma unroll
      for (int t = 0; t < NT; t++)
#pragma unroll
        for (int i = 0; i < 2; i++) {
          const double ht = d[t][i];
          const double x = ht - u[t][i];
          const double hn = (a.prox == CSTF_PROX_IDENTITY) ? x : (x > 0.0 ? x : 0.0);
          const double un = (u[t][i] + hn) - ht;
          const double e1 = hn - ht, e2 = hn - h[t][i];
          pr = fma(e1, e1, pr); ps = fma(e2, e2, ps); ph = fma(hn, hn, ph); pu = fma(un, un, pu);
          h[t][i] = hn;
          u[t][i] = un;
        }
      double* sj = sacc + (size_t)j * 4 * kThreads + tid;
      sj[0] += pr; sj[kThreads] += ps; sj[2 * kThreads] += ph; sj[3 * kThreads] += pu;
    }
    if (a.Hout && rok) {
#pragma unroll
      for (int t = 0; t < NT; t++) {
        const int col = 8 * t + 2 * q;
        if (full) {
          __stcs(reinterpret_cast<double2*>(a.Hout + base + col), make_double2(h[t][0], h[t][1]));
          __stcs(reinterpret_cast<double2*>(a.Uout + base + col), make_double2(u[t][0], u[t][1]));
        } else {
#pragma unroll
          for (int i = 0; i < 2; i++)
            if (col + i < R) { a.Hout[base + col + i] = h[t][i]; a.Uout[base + col + i] = u[t][i]; }
        }
      }
    }
  }
  __syncthreads();
  // fixed-order CTA reduction of the per-thread slots
  for (int x = tid; x < kiters * 4; x += kThreads) {
    const double* p = sacc + (size_t)x * kThreads;
    double s = 0.0;
    for (int k = 0; k < kThreads; k++) s += p[k];
    const int j = x >> 2, w = x & 3;
    a.slots[((size_t)j * gridDim.x + blockIdx.x) * 4 + w] = s;
  }
}

// Generic form for any R <= 128: one CTA row at a time, thread = column,
// Inv column in registers-from-smem.  Same per-element arithmetic order.
__global__ void __launch_bounds__(128) k_admm_generic(KArgs a) {
  extern __shared__ double smem[];
  double* sinv = smem;                       // [R][R]
  double* st = smem + (size_t)a.R * a.R;     // [R] T of the current row
  double* sacc = st + 128;                   // [kiters][4][128]
  const int tid = threadIdx.x;
  const int R = a.R;
  const bool skip = *a.flag != 0;
  const double rho = a.scal[0];
  const int kiters = a.kiters;
  for (int x = tid; x < R * R; x += blockDim.x) sinv[x] = a.inv[x];
  for (int x = tid; x < kiters * 4 * 128; x += blockDim.x) sacc[x] = 0.0;
  __syncthreads();
  const bool cok = tid < R;
  const double hsc = (a.hscale && cok) ? a.hscale[tid] : 1.0;
  for (int64_t row = skip ? a.I : blockIdx.x; row < a.I; row += gridDim.x) {
    const size_t base = (size_t)row * R;
    double m = cok ? a.M[base + tid] : 0.0;
    double h = cok ? a.H[base + tid] * hsc : 0.0;
    double u = cok ? a.U[base + tid] : 0.0;
    for (int j = 0; j < kiters; j++) {
      if (cok) st[tid] = fma(rho, h + u, m);
      __syncthreads();
      double ht = 0.0;
      if (cok)
        for (int k = 0; k < R; k++) ht = fma(st[k], sinv[k * R + tid], ht);
      __syncthreads();
      const double x = ht - u;
      const double hn = (a.prox == CSTF_PROX_IDENTITY) ? x : (x > 0.0 ? x : 0.0);
      const double un = (u + hn) - ht;
      const double e1 = hn - ht, e2 = hn - h;
      if (cok) {
        double* sj = sacc + (size_t)j * 4 * 128 + tid;
        sj[0] = fma(e1, e1, sj[0]); sj[128] = fma(e2, e2, sj[128]);
        sj[256] = fma(hn, hn, sj[256]); sj[384] = fma(un, un, sj[384]);
        h = hn;
        u = un;
      }
    }
    if (a.Hout && cok) { a.Hout[base + tid] = h; a.Uout[base + tid] = u; }
  }
  __syncthreads();
  for (int x = tid; x < kiters * 4; x += blockDim.x) {
    const double* p = sacc + (size_t)x * 128;
    double s = 0.0;
    for (int k = 0; k < 128; k++) s += p[k];
    const int j = x >> 2, w = x & 3;
    a.slots[((size_t)j * gridDim.x + blockIdx.x) * 4 + w] = s;
  }
}

// sums[j0 + j][w] = sum over CTAs (fixed order) of slots[j][cta][w]
__global__ void k_admm_sum(const double* __restrict__ slots, int nblocks, int kiters, int j0,
                           double* __restrict__ sums) {
  for (int x = threadIdx.x; x < kiters * 4; x += blockDim.x) {
    const int j = x >> 2, w = x & 3;
    double s = 0.0;
    for (int b = 0; b < nblocks; b++) s += slots[((size_t)j * nblocks + b) * 4 + w];
    sums[(size_t)(j0 + j) * 4 + w] = s;
  }
}

// Stop decision over iterations [j0, j0 + k): first j with r < tol nH and s < tol nU (D3),
// or the last allowed iteration.  dec[0] = decided iteration count (0 = undecided),
// dec[1] = flags (2 = non-finite).  stats out: iters, rho, r, s, nH, nU.
__global__ void k_admm_decide(const double* __restrict__ sums, int j0, int k, int max_iter, double tol,
                              const double* __restrict__ scal, int* __restrict__ flag,
                              double* __restrict__ out) {
  if (threadIdx.x != 0) return;
  int decided = 0;
  for (int j = j0; j < j0 + k; j++) {
    const double r = sums[j * 4 + 0], s = sums[j * 4 + 1], nH = sums[j * 4 + 2], nU = sums[j * 4 + 3];
    if (!isfinite(r) || !isfinite(s) || !isfinite(nH) || !isfinite(nU)) {
      atomicOr(flag, 2);
      decided = j + 1;
      break;
    }
    if ((tol > 0.0 && r < tol * nH && s < tol * nU) || j + 1 == max_iter) {
      decided = j + 1;
      break;
    }
  }
  out[0] = decided;
  if (decided) {
    const int j = decided - 1;
    out[1] = scal[0];
    out[2] = sums[j * 4 + 0]; out[3] = sums[j * 4 + 1]; out[4] = sums[j * 4 + 2]; out[5] = sums[j * 4 + 3];
  }
}

struct Workspace {
  DevBuf slots, sums, out, hs[2], us[2];
  double* host_out = nullptr;
};
Workspace& ws() {
  static thread_local Workspace w[64];
  int dev = 0;
  cudaGetDevice(&dev);
  Workspace& r = w[dev & 63];
  if (!r.host_out) cudaMallocHost(&r.host_out, 16 * sizeof(double));
  return r;
}

template <int RP, bool REG>
cstf_status launch_dmma_t(const KArgs& k, int grid, cudaStream_t st) {
  const size_t smem = (size_t)kMaxK * 4 * kThreads * 8 + (REG ? 0 : (size_t)2 * (RP / 8) * (RP / 8) * 32 * 8);
  static bool attr = false;
  if (!attr) {
    CSTF_CUDA(cudaFuncSetAttribute(k_admm_dmma<RP, REG>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    attr = true;
  }
  k_admm_dmma<RP, REG><<<grid, kThreads, smem, st>>>(k);
  CSTF_LAUNCHED();
  return CSTF_OK;
}

int grid_for_dmma(int RP, int64_t I) {
  // persistent: up to (SMs x CTAs/SM); fewer when there are few row groups
  const int sms = device_info().sms;
  const int per_sm = RP <= 32 ? 3 : 2;
  const int64_t groups = (I + 7) / 8;
  int64_t g = (groups + 3) / 4;
  int64_t cap = (int64_t)sms * per_sm;
  if (g > cap) g = cap;
  return (int)(g < 1 ? 1 : g);
}

cstf_status launch_kernel(const KArgs& k, int& grid, cudaStream_t st) {
  const int R = k.R;
  const int RP = (R + 7) & ~7;
  if (RP <= 64) {
    grid = grid_for_dmma(RP, k.I);
    switch (RP) {
      case 8: return launch_dmma_t<8, true>(k, grid, st);
      case 16: return launch_dmma_t<16, true>(k, grid, st);
      case 24: return launch_dmma_t<24, true>(k, grid, st);
      case 32: return launch_dmma_t<32, true>(k, grid, st);
      case 40: return launch_dmma_t<40, false>(k, grid, st);
      case 48: return launch_dmma_t<48, false>(k, grid, st);
      case 56: return launch_dmma_t<56, false>(k, grid, st);
      case 64: return launch_dmma_t<64, false>(k, grid, st);
    }
  }
  grid = (int)std::min<int64_t>(std::max<int64_t>(k.I, 1), (int64_t)device_info().sms * 8);
  const size_t smem = (size_t)R * R * 8 + 128 * 8 + (size_t)kMaxK * 4 * 128 * 8;
  static bool attr = false;
  if (!attr) {
    CSTF_CUDA(cudaFuncSetAttribute(k_admm_generic, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                   (int)((size_t)128 * 128 * 8 + 128 * 8 + (size_t)kMaxK * 4 * 128 * 8)));
    attr = true;
  }
  k_admm_generic<<<grid, 128, smem, st>>>(k);
  CSTF_LAUNCHED();
  return CSTF_OK;
}

}  // namespace

// Runs one ADMM update.  tol == 0: chunks of up to kMaxK iterations in place,
// no host round trip until the end.  tol > 0: each chunk runs speculatively
// into scratch buffers, the device decides the stop iteration, and the chunk
// is replayed exactly (same arithmetic) up to it when it ends early.
cstf_status admm_run(const AdmmArgs& A, const cstf_comm* comm, cudaStream_t st,
                     cstf_admm_stats* stats, int* iters_out, int64_t* launches) {
  Workspace& w = ws();
  const int R = A.R;
  const int64_t I = A.I;
  const int kchunk = (A.variant == CSTF_ADMM_STREAMING) ? 1 : kMaxK;
  const int maxgrid = device_info().sms * 8;
  CSTF_TRY(w.slots.ensure((size_t)kMaxK * maxgrid * 4 * 8));
  CSTF_TRY(w.sums.ensure((size_t)A.max_iter * 4 * 8));
  CSTF_TRY(w.out.ensure(16 * 8));
  int64_t nl = 0;
  KArgs k;
  k.M = A.M;
  k.I = I;
  k.R = R;
  k.inv = A.inv;
  k.scal = A.scal;
  k.flag = A.flag;
  k.prox = A.prox;
  k.slots = w.slots.as<double>();
  const bool spec = A.tol > 0.0;
  if (spec) {
    for (int b = 0; b < 2; b++) {
      CSTF_TRY(w.hs[b].ensure((size_t)I * R * 8));
      CSTF_TRY(w.us[b].ensure((size_t)I * R * 8));
    }
  }
  const double* curH = A.H;
  const double* curU = A.U;
  const double* cur_scale = A.hscale;
  int pp = 0;
  int decided = 0;
  for (int j0 = 0; j0 < A.max_iter;) {
    const int kk = std::min(kchunk, A.max_iter - j0);
    k.H = curH;
    k.U = curU;
    k.hscale = cur_scale;
    k.kiters = kk;
    if (spec && kchunk > 1) {
      k.Hout = w.hs[pp].as<double>();
      k.Uout = w.us[pp].as<double>();
    } else {
      k.Hout = A.H;   // in place
      k.Uout = A.U;
    }
    int grid = 0;
    CSTF_TRY(launch_kernel(k, grid, st));
    k_admm_sum<<<1, 64, 0, st>>>(k.slots, grid, kk, j0, w.sums.as<double>());
    CSTF_LAUNCHED();
    nl += 2;
    if (comm_nranks(comm) > 1) CSTF_TRY(comm_allreduce_f64(comm, w.sums.as<double>() + (size_t)j0 * 4, (size_t)kk * 4, st));
    if (!spec) {
      j0 += kk;
      curH = A.H; curU = A.U; cur_scale = nullptr;
      if (j0 >= A.max_iter) {
        k_admm_decide<<<1, 32, 0, st>>>(w.sums.as<double>(), A.max_iter - 1, 1, A.max_iter, 0.0, A.scal,
                                         A.flag, w.out.as<double>());
        CSTF_LAUNCHED();
        nl++;
        decided = A.max_iter;
      }
      continue;
    }
    k_admm_decide<<<1, 32, 0, st>>>(w.sums.as<double>(), j0, kk, A.max_iter, A.tol, A.scal, A.flag,
                                     w.out.as<double>());
    CSTF_LAUNCHED();
    nl++;
    CSTF_CUDA(cudaMemcpyAsync(w.host_out, w.out.p, 6 * 8, cudaMemcpyDeviceToHost, st));
    CSTF_CUDA(cudaStreamSynchronize(st));
    const int dj = (int)w.host_out[0];
    if (dj == 0) {               // not decided in this chunk: continue from its end state
      if (kchunk > 1) {
        curH = w.hs[pp].as<double>();
        curU = w.us[pp].as<double>();
        pp ^= 1;
      } else {
        curH = A.H; curU = A.U;
      }
      cur_scale = nullptr;
      j0 += kk;
      continue;
    }
    decided = dj;
    if (kchunk > 1) {
      if (dj == j0 + kk) {       // stop at the chunk's last pass: its end state is the answer
        CSTF_CUDA(cudaMemcpyAsync(A.H, w.hs[pp].p, (size_t)I * R * 8, cudaMemcpyDeviceToDevice, st));
        CSTF_CUDA(cudaMemcpyAsync(A.U, w.us[pp].p, (size_t)I * R * 8, cudaMemcpyDeviceToDevice, st));
      } else {                   // exact replay of the chunk up to the decided pass
        k.H = curH; k.U = curU; k.hscale = cur_scale;
        k.kiters = dj - j0;
        k.Hout = A.H; k.Uout = A.U;
        CSTF_TRY(launch_kernel(k, grid, st));
        nl++;
      }
    }
    break;
  }
  if (launches) *launches += nl;
  if (iters_out) *iters_out = decided;
  if (stats) {
    if (!spec) {
      CSTF_CUDA(cudaMemcpyAsync(w.host_out, w.out.p, 6 * 8, cudaMemcpyDeviceToHost, st));
      CSTF_CUDA(cudaStreamSynchronize(st));
    }
    stats->iters = decided;
    stats->rho = w.host_out[1];
    stats->r_primal = w.host_out[2];
    stats->s_dual = w.host_out[3];
    stats->normH2 = w.host_out[4];
    stats->normU2 = w.host_out[5];
  }
  return CSTF_OK;
}

}  // namespace cstf
