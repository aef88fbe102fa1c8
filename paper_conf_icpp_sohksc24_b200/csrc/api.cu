// extern "C" entry points of libcstf (include/cstf.h) and the Alg. 1 driver.
#include <cstdlib>
#include <cstring>
#include <vector>

#include "internal.h"

using namespace cstf;

namespace {

cudaStream_t S(void* s) { return static_cast<cudaStream_t>(s); }

// dst[lab[i]] = src[i] (to_internal) or dst[i] = src[lab[i]] (from internal), rows of R doubles
__global__ void k_relabel_rows(const double* __restrict__ src, const int32_t* __restrict__ lab, int64_t I, int R,
                               double* __restrict__ dst, int to_internal) {
  const int64_t n = I * R;
  for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < n; x += (int64_t)gridDim.x * blockDim.x) {
    const int64_t i = x / R, c = x % R;
    const int64_t l = lab[i];
    if (to_internal) dst[l * R + c] = src[x];
    else dst[x] = src[l * R + c];
  }
}

cstf_status relabel_rows(const double* src, const int32_t* lab, int64_t I, int R, double* dst, int to_internal,
                         cudaStream_t st) {
  if (I * R == 0) return CSTF_OK;
  const int g = (int)std::min<int64_t>((I * R + 255) / 256, (int64_t)device_info().sms * 16);
  k_relabel_rows<<<g, 256, 0, st>>>(src, lab, I, R, dst, to_internal);
  CSTF_LAUNCHED();
  return CSTF_OK;
}

bool rank_ok(int R) { return R >= 1 && R <= 128; }

// Device-side scratch of one factorize / admm_update call, cached per device.
struct DriverWs {
  DevBuf grams, lam, inv, scal, flag, fitbuf, fits, M, U, hostfac, Fi[8], S, stage;
  cudaStream_t copy = nullptr;   // host <-> device factor transfers of cstf_factorize_host
  cudaEvent_t ev_in[8] = {nullptr}, ev_out[8] = {nullptr};
  // distributed: all internal factor replicas in one allocation, mapped by the
  // other ranks through CUDA IPC (NVLink peer memory) for the fused all-gather
  DevBuf facall, xchg, agreebuf;
  uint64_t facall_gen = 0;       // bumped on every facall (re)allocation: equal on all ranks
  uint64_t ipc_gen = ~0ull;      // facall_gen the peer mappings were made for
  const cstf_comm* ipc_comm = nullptr;
  int ipc_state = 0;             // 0 none, 1 peers mapped, 2 agreed: no peer stores
  double* ipc_peer[8] = {nullptr};
  double* host_small = nullptr;  // pinned: fit, flags
  cudaStream_t side = nullptr;   // the R x R step of a mode overlaps its MTTKRP
  cudaEvent_t fork = nullptr, join = nullptr;
};
DriverWs& dws() {
  static thread_local DriverWs w[64];
  int dev = 0;
  cudaGetDevice(&dev);
  DriverWs& r = w[dev & 63];
  if (!r.host_small) cudaMallocHost(&r.host_small, 64 * sizeof(double));
  if (!r.side) {
    cudaStreamCreateWithFlags(&r.side, cudaStreamNonBlocking);
    cudaEventCreateWithFlags(&r.fork, cudaEventDisableTiming);
    cudaEventCreateWithFlags(&r.join, cudaEventDisableTiming);
    cudaStreamCreateWithFlags(&r.copy, cudaStreamNonBlocking);
    for (int n = 0; n < 8; n++) {
      cudaEventCreateWithFlags(&r.ev_in[n], cudaEventDisableTiming);
      cudaEventCreateWithFlags(&r.ev_out[n], cudaEventDisableTiming);
    }
  }
  return r;
}

// Agree on a status across ranks (a collective call returns the same
// status on every rank).  Each rank contributes a one-hot vector of its status; the
// all-reduced vector names every status that occurred, and all ranks return the
// largest code.  A rank whose own call succeeded reports which status another rank hit.
cstf_status agree(DriverWs& w, const cstf_comm* comm, cstf_status local, cudaStream_t st) {
  if (comm_nranks(comm) <= 1) return local;
  if (w.agreebuf.ensure(8 * 8) != CSTF_OK) return local;      // cannot agree: report the local status
  double v[8] = {0};
  v[(int)local & 7] = 1.0;
  double* d = w.agreebuf.as<double>();
  if (cudaMemcpyAsync(d, v, sizeof(v), cudaMemcpyHostToDevice, st) != cudaSuccess) return local;
  if (comm_allreduce_f64(comm, d, 8, st) != CSTF_OK) return local;
  if (cudaMemcpyAsync(v, d, sizeof(v), cudaMemcpyDeviceToHost, st) != cudaSuccess) return local;
  if (cudaStreamSynchronize(st) != cudaSuccess) return local;
  int worst = 0;
  for (int k = 1; k < 8; k++)
    if (v[k] > 0.0) worst = k;
  if (worst == 0 || worst == (int)local) return local;
  return fail((cstf_status)worst, std::string("another rank failed with ") + cstf_status_string((cstf_status)worst) +
                                      (local != CSTF_OK ? std::string(" (this rank: ") + cstf_status_string(local) + ")"
                                                        : std::string()));
}

// Map every other rank's factor replicas (CUDA IPC handles exchanged through the
// communicator).  Collective on EVERY call: each rank says whether its mappings are
// stale (facall re-allocated, other communicator, never decided); if any rank is
// stale all ranks drop their mappings and redo the exchange, so no rank skips a
// collective another rank enters, and no mapping outlives the allocation it was made
// for.  Before opening a handle, the peer's device (PCI bus id) must be visible and
// peer-accessible from ours (or be our own device).  Returns the same answer on every
// rank: true only if every rank mapped every peer.
bool open_peers(DriverWs& w, const cstf_comm* comm, cudaStream_t st) {
  const int P = comm_nranks(comm), me = comm_rank(comm);
  static_assert(sizeof(cudaIpcMemHandle_t) == 64, "IPC handle size");
  constexpr int kW = 10;                       // doubles per rank: 64-byte handle + 16-byte PCI bus id
  if (w.xchg.ensure((size_t)(kW * P + kW) * 8) != CSTF_OK) return false;
  double* d = w.xchg.as<double>();
  const bool stale = !(w.ipc_state != 0 && w.ipc_gen == w.facall_gen && w.ipc_comm == comm);
  double flag = stale ? 1.0 : 0.0;
  if (cudaMemcpyAsync(d, &flag, 8, cudaMemcpyHostToDevice, st) != cudaSuccess) return false;
  if (comm_allreduce_f64(comm, d, 1, st) != CSTF_OK) return false;
  if (cudaMemcpyAsync(&flag, d, 8, cudaMemcpyDeviceToHost, st) != cudaSuccess) return false;
  if (cudaStreamSynchronize(st) != cudaSuccess) return false;
  if (flag == 0.0) return w.ipc_state == 1;    // every rank fresh: the last (agreed) decision stands
  for (int r = 0; r < 8; r++)
    if (w.ipc_peer[r]) { cudaIpcCloseMemHandle(w.ipc_peer[r]); w.ipc_peer[r] = nullptr; }
  w.ipc_state = 0;
  const char* env = getenv("CSTF_PEER_STORE");
  double ok = (P <= 8 && !(env && atoi(env) == 0)) ? 1.0 : 0.0;
  unsigned char mine[kW * 8];
  memset(mine, 0, sizeof(mine));
  int mydev = 0;
  cudaGetDevice(&mydev);
  if (ok > 0 && cudaIpcGetMemHandle(reinterpret_cast<cudaIpcMemHandle_t*>(mine), w.facall.p) != cudaSuccess) {
    cudaGetLastError();
    ok = 0;
  }
  if (cudaDeviceGetPCIBusId(reinterpret_cast<char*>(mine) + 64, 16, mydev) != cudaSuccess) {
    cudaGetLastError();
    ok = 0;
  }
  if (cudaMemcpyAsync(d + kW * P, mine, sizeof(mine), cudaMemcpyHostToDevice, st) != cudaSuccess) return false;
  if (comm_allgather_f64(comm, d + kW * P, d, kW, st) != CSTF_OK) return false;
  std::vector<unsigned char> all((size_t)P * kW * 8);
  if (cudaMemcpyAsync(all.data(), d, all.size(), cudaMemcpyDeviceToHost, st) != cudaSuccess) return false;
  if (cudaStreamSynchronize(st) != cudaSuccess) return false;
  for (int r = 0; r < P && ok > 0; r++) {
    if (r == me) continue;
    const unsigned char* rec = all.data() + (size_t)r * kW * 8;
    char bus[17];
    memcpy(bus, rec + 64, 16);
    bus[16] = 0;
    int pdev = -1, can = 0;
    if (cudaDeviceGetByPCIBusId(&pdev, bus) != cudaSuccess) {      // peer GPU not visible here
      cudaGetLastError();
      ok = 0;
      break;
    }
    if (pdev != mydev && (cudaDeviceCanAccessPeer(&can, mydev, pdev) != cudaSuccess || !can)) {
      cudaGetLastError();
      ok = 0;
      break;
    }
    cudaIpcMemHandle_t h;
    memcpy(&h, rec, 64);
    void* ptr = nullptr;
    if (cudaIpcOpenMemHandle(&ptr, h, cudaIpcMemLazyEnablePeerAccess) != cudaSuccess) {
      cudaGetLastError();
      ok = 0;
    } else {
      w.ipc_peer[r] = static_cast<double*>(ptr);
    }
  }
  // consensus: every rank uses peer stores or none does
  double fails = ok > 0 ? 0.0 : 1.0;
  if (cudaMemcpyAsync(d, &fails, 8, cudaMemcpyHostToDevice, st) != cudaSuccess) return false;
  if (comm_allreduce_f64(comm, d, 1, st) != CSTF_OK) return false;
  if (cudaMemcpyAsync(&fails, d, 8, cudaMemcpyDeviceToHost, st) != cudaSuccess) return false;
  if (cudaStreamSynchronize(st) != cudaSuccess) return false;
  w.ipc_gen = w.facall_gen;
  w.ipc_comm = comm;
  if (fails > 0) {
    for (int r = 0; r < 8; r++)
      if (w.ipc_peer[r]) { cudaIpcCloseMemHandle(w.ipc_peer[r]); w.ipc_peer[r] = nullptr; }
    w.ipc_state = 2;
    return false;
  }
  w.ipc_state = 1;
  return true;
}

cstf_status check_flag(const int* d_flag, cudaStream_t st) {
  int f = 0;
  CSTF_CUDA(cudaMemcpyAsync(&f, d_flag, 4, cudaMemcpyDeviceToHost, st));
  CSTF_CUDA(cudaStreamSynchronize(st));
  if (f & 1) return fail(CSTF_ERR_NOT_SPD, "S + rho I is not positive definite (rho <= 0 or pivot <= 0)");
  if (f & 2) return fail(CSTF_ERR_NUMERIC, "non-finite ADMM residual or fit");
  return CSTF_OK;
}

struct PhaseTimer {
  bool on = false;
  cudaStream_t st = nullptr;
  std::vector<cudaEvent_t> ev;
  std::vector<int> mode, phase;   // segment k: ev[2k] .. ev[2k+1]
  std::vector<int64_t> l0;
  double* phase_ms = nullptr;
  double* mode_phase_ms = nullptr;
  int64_t* mode_launches = nullptr;
  int nseg = 0;
  int64_t launch_mark = 0;
  ~PhaseTimer() { for (auto e : ev) cudaEventDestroy(e); }
  void begin(int m, int p) {
    launch_mark = cstf_kernel_launch_count();
    if (!on) return;
    if ((size_t)(2 * nseg + 2) > ev.size()) {
      for (int k = 0; k < 2; k++) { cudaEvent_t e; cudaEventCreate(&e); ev.push_back(e); }
    }
    cudaEventRecord(ev[2 * nseg], st);
    if ((size_t)nseg >= mode.size()) { mode.push_back(m); phase.push_back(p); }
    else { mode[nseg] = m; phase[nseg] = p; }
  }
  void end(int m, int p) {
    if (mode_launches) mode_launches[m * CSTF_NUM_PHASES + p] += cstf_kernel_launch_count() - launch_mark;
    if (!on) return;
    cudaEventRecord(ev[2 * nseg + 1], st);
    nseg++;
  }
  // after a stream sync: accumulate and reset
  void collect() {
    for (int k = 0; k < nseg; k++) {
      float ms = 0.f;
      cudaEventElapsedTime(&ms, ev[2 * k], ev[2 * k + 1]);
      if (phase_ms) phase_ms[phase[k]] += ms;
      if (mode_phase_ms) mode_phase_ms[mode[k] * CSTF_NUM_PHASES + phase[k]] += ms;
    }
    nseg = 0;
  }
};

// Host I/O of cstf_factorize_host overlapped with the computation (single GPU):
// host_in[n] -> d_factors[n] on the copy stream, in the order the first outer
// iteration needs them (factor 0 only before the first ADMM update); with a
// fixed number of outer iterations, each final factor is normalised into a
// staging copy right after its last update and copied to host_out[n] while the
// later modes compute.
struct HostIO {
  double* const* in = nullptr;
  double* const* out = nullptr;
};

cstf_status factorize_impl(const cstf_tensor* X, const cstf_opts* o, const cstf_comm* comm,
                           double* const* d_factors, double* d_lambda, cstf_report* rep,
                           cudaStream_t st, const HostIO* hio = nullptr) {
  const int N = X->N;
  const int R = o->R;
  const bool dist = X->partitioned;
  DriverWs& w = dws();
  // Distributed: every rank keeps full factors in the
  // internal (relabelled, zero-padded) row order; its own rows are the slice
  // [rank*B_n, (rank+1)*B_n).  Single GPU: the caller's buffers, all rows local.
  std::vector<double*> fac(N), U(N);
  std::vector<int64_t> Ifull(N), Iloc(N), off(N), facoff(N);
  int64_t Imax = 0, Usum = 0;
  const bool sync_each = o->fit_tol > 0.0;
  // Setup: validation and every allocation.  Distributed, its status is agreed over
  // the ranks before the first collective of the algorithm, so a rank that fails
  // here (bad argument, out of memory) makes every rank return the same status
  // instead of leaving the others blocked in a collective.
  auto setup = [&]() -> cstf_status {
    if (!rank_ok(R)) return fail(CSTF_ERR_UNSUPPORTED, "R must be in [1, 128]");
    if (o->outer_iters < 1 || o->admm.max_iter < 1) return fail(CSTF_ERR_INVALID_ARG, "outer_iters/max_iter < 1");
    if (o->admm.prox < CSTF_PROX_NONNEG || o->admm.prox > CSTF_PROX_BOX || !(o->admm.alpha >= 0.0) ||
        (o->admm.prox == CSTF_PROX_BOX && !(o->admm.alpha > 0.0)))
      return fail(CSTF_ERR_INVALID_ARG, "unknown prox or alpha < 0");
    if (o->update < CSTF_UPDATE_ADMM || o->update > CSTF_UPDATE_MU) return fail(CSTF_ERR_INVALID_ARG, "unknown update");
    if (o->update == CSTF_UPDATE_MU && R > 64) return fail(CSTF_ERR_UNSUPPORTED, "MU update for R > 64");
    if ((comm != nullptr) != dist || comm_nranks(comm) != X->nranks || (dist && comm_rank(comm) != X->rank))
      return fail(CSTF_ERR_INVALID_ARG, "comm does not match the tensor's partition");
    for (int n = 0; n < N; n++)
      if (!d_factors[n]) return fail(CSTF_ERR_INVALID_ARG, "factor pointer is NULL");
    if (dist) {
      const char* inj = getenv("CSTF_TEST_FAIL_RANK");     // tests: one rank fails its setup
      if (inj && atoi(inj) == X->rank) return fail(CSTF_ERR_OUT_OF_MEMORY, "injected setup failure (CSTF_TEST_FAIL_RANK)");
    }
    if (dist) {                         // one allocation for all replicas (IPC-mappable)
      int64_t tot = 0;
      for (int n = 0; n < N; n++) {
        facoff[n] = tot;
        tot += ((int64_t)X->nranks * X->rows_per_rank[n] * R + 31) / 32 * 32;
      }
      const void* before = w.facall.p;
      const size_t bytes_before = w.facall.bytes;
      CSTF_TRY(w.facall.ensure((size_t)tot * 8));
      // the size depends only on global sizes, so every rank re-allocates in the same call
      if (w.facall.p != before || w.facall.bytes != bytes_before) w.facall_gen++;
    }
    for (int n = 0; n < N; n++) {
      if (dist) {
        const int64_t B = X->rows_per_rank[n];
        Ifull[n] = (int64_t)X->nranks * B;
        Iloc[n] = B;
        off[n] = (int64_t)X->rank * B * R;
        fac[n] = w.facall.as<double>() + facoff[n];
        CSTF_CUDA(cudaMemsetAsync(fac[n], 0, (size_t)Ifull[n] * R * 8, st));
        CSTF_TRY(relabel_rows(d_factors[n], X->relabel[n].as<int32_t>(), X->dims[n], R, fac[n], 1, st));
      } else {
        Ifull[n] = Iloc[n] = X->dims[n];
        off[n] = 0;
        fac[n] = d_factors[n];
      }
    }
    for (int n = 0; n < N; n++) { Imax = std::max(Imax, Iloc[n]); Usum += Iloc[n] * R; }
    CSTF_TRY(w.grams.ensure((size_t)N * R * R * 8));
    CSTF_TRY(w.lam.ensure((size_t)(N + 1) * R * 8));     // + R scratch for the initial column norms
    CSTF_TRY(w.inv.ensure((size_t)R * R * 8));
    CSTF_TRY(w.S.ensure((size_t)R * R * 8));
    CSTF_TRY(w.scal.ensure((size_t)(8 + 2 * R) * 8));
    CSTF_TRY(w.flag.ensure(64));
    CSTF_TRY(w.fitbuf.ensure(300 * 8));
    // with a fixed number of outer iterations (fit_tol = 0) the loop runs without a
    // host round trip; the fits are collected at the end
    if (!sync_each) CSTF_TRY(w.fits.ensure((size_t)2 * o->outer_iters * 8));
    CSTF_TRY(w.M.ensure((size_t)Imax * R * 8));
    CSTF_TRY(w.U.ensure((size_t)Usum * 8));
    int64_t uo = 0;
    for (int n = 0; n < N; n++) { U[n] = w.U.as<double>() + uo; uo += Iloc[n] * R; }
    CSTF_CUDA(cudaMemsetAsync(w.flag.p, 0, 4, st));
    CSTF_CUDA(cudaMemsetAsync(w.U.p, 0, (size_t)Usum * 8, st));
    return CSTF_OK;
  };
  {
    cstf_status s0 = setup();
    if (dist) s0 = agree(w, comm, s0, st);
    if (s0 != CSTF_OK) return s0;
  }
  // f4: fused all-gather through peer stores from the ADMM epilogue (falls back to
  // the NCCL / host all-gather when IPC mapping is unavailable or disabled)
  const bool peers = dist && open_peers(w, comm, st);
  // hot-row tables (single GPU, factors >> L2): persisting set-aside for the whole call,
  // released (and the caller's limit restored) on every return path
  struct HotGuard {
    L2Persist p;
    cudaStream_t st;
    ~HotGuard() {
      if (p.active) {
        cudaStreamSynchronize(st);
        hot_persist_end(p);
      }
    }
  } hotg;
  hotg.st = st;
  CSTF_TRY(hot_persist_begin(X, hotg.p));
  double* G = w.grams.as<double>();
  double* lam = w.lam.as<double>();
  double* lam_scratch = lam + (size_t)N * R;
  double* M = w.M.as<double>();
  int* flag = w.flag.as<int>();
  const bool hin = hio && hio->in && !dist;
  const bool hout = hio && hio->out && !dist && o->fit_tol <= 0.0;
  if (hin) {                         // factors 1..N-1 first, factor 0 last (needed only by ADMM(0))
    CSTF_CUDA(cudaEventRecord(w.fork, st));
    CSTF_CUDA(cudaStreamWaitEvent(w.copy, w.fork, 0));
    for (int k = 1; k <= N; k++) {
      const int n = k % N;
      CSTF_CUDA(cudaMemcpyAsync(fac[n], hio->in[n], (size_t)Ifull[n] * R * 8, cudaMemcpyHostToDevice, w.copy));
      CSTF_CUDA(cudaEventRecord(w.ev_in[n], w.copy));
    }
  }
  // init (Alg. 1 l.1-5; readings D6): normalise, lambda = 1, G = H^T H
  // (the column norms go to a scratch vector, never to lam: with host input, init of
  // factor 0 runs after MTTKRP(0) while the side stream's Cholesky of mode 0 reads
  // lam[0..R), which is set to 1 before the loop and not written again here)
  auto init_factor = [&](int n, bool set_lam) -> cstf_status {
    double* Gn = G + (size_t)n * R * R;
    if (hin) CSTF_CUDA(cudaStreamWaitEvent(st, w.ev_in[n], 0));
    CSTF_TRY(gram_raw(fac[n], Ifull[n], R, Gn, st));
    if (o->normalize_init) CSTF_TRY(normalize_from_gram(fac[n], Ifull[n], R, Gn, lam_scratch, st));
    return set_lam ? fill(lam + n * R, R, 1.0, st) : CSTF_OK;
  };
  for (int n = 0; n < N; n++) {      // factors are replicated: redundant, no communication
    if (hin && n == 0) {             // deferred: after MTTKRP(0) is queued
      CSTF_TRY(fill(lam, R, 1.0, st));
      continue;
    }
    CSTF_TRY(init_factor(n, true));
    CSTF_TRY(hot_refresh(X, n, fac[n], R, st));     // (no-op without hot rows)
  }
  if (peers) {   // no rank may peer-store into a replica another rank is still initialising / reading
    CSTF_TRY(comm_allreduce_f64(comm, w.xchg.as<double>(), 1, st));
  }
  std::vector<int64_t> stage_off(N, 0);
  if (hout) {
    int64_t so = 0;
    for (int n = 0; n < N; n++) { stage_off[n] = so; so += Ifull[n] * R; }
    CSTF_TRY(w.stage.ensure((size_t)so * 8));
  }
  PhaseTimer tm;
  tm.on = o->timing != 0;
  tm.st = st;
  if (rep) {
    tm.phase_ms = rep->phase_ms;
    tm.mode_phase_ms = rep->mode_phase_ms;
    tm.mode_launches = rep->mode_launches;
    if (rep->phase_ms) for (int p = 0; p < CSTF_NUM_PHASES; p++) rep->phase_ms[p] = 0.0;
    if (rep->mode_phase_ms) for (int p = 0; p < N * CSTF_NUM_PHASES; p++) rep->mode_phase_ms[p] = 0.0;
    if (rep->mode_launches) for (int p = 0; p < N * CSTF_NUM_PHASES; p++) rep->mode_launches[p] = 0;
    rep->outer_done = 0;
  }
  // Lazy normalisation: d_factors hold the raw ADMM output
  // H_raw = H^(n) diag(lambda^(n)); the normalised factor is never formed inside
  // the loop.  MTTKRP of the raw factors is rescaled per column on the ADMM
  // load (mscale = prod_{k != n} 1/lambda_k), the scaled warm start (D4) is
  // H_raw itself, the Grams kept are those of the normalised factors, and the
  // factors are normalised once at the end.
  CSTF_TRY(w.scal.ensure((size_t)(8 + 2 * R) * 8));
  double* colscale = w.scal.as<double>() + 8;           // [2R]: mscale, 1/lambda_n
  double fit_prev = 0.0;
  for (int t = 0; t < o->outer_iters; t++) {
    for (int n = 0; n < N; n++) {
      const int64_t I = Iloc[n];
      double* Hn = fac[n] + off[n];     // this rank's rows of the raw factor
      double* Gn = G + (size_t)n * R * R;
      // a1 + a3 + a4 (S, rho, Cholesky, Inv: one CTA) run on a side stream,
      // concurrently with a2 (MTTKRP) which does not depend on them
      CSTF_CUDA(cudaEventRecord(w.fork, st));
      CSTF_CUDA(cudaStreamWaitEvent(w.side, w.fork, 0));
      CSTF_TRY(chol_inverse(nullptr, G, N, n, R, o->admm.rho, w.inv.as<double>(), w.scal.as<double>(), flag,
                            w.side, lam, colscale, w.S.as<double>()));
      CSTF_CUDA(cudaEventRecord(w.join, w.side));
      // a2: MTTKRP of the raw factors (MTTKRP phase = both, overlapped)
      tm.begin(n, CSTF_PHASE_MTTKRP);
      CSTF_TRY(mttkrp(X, n, R, fac.data(), M, st, nullptr, /*hot_fresh=*/true));
      if (hin && t == 0 && n == 0) CSTF_TRY(init_factor(0, false));   // its copy overlapped MTTKRP(0)
      CSTF_CUDA(cudaStreamWaitEvent(st, w.join, 0));
      tm.end(n, CSTF_PHASE_MTTKRP);
      // a5: ADMM on M diag(mscale); warm start H_raw (D4) or the normalised H (literal)
      tm.begin(n, CSTF_PHASE_UPDATE);
      AdmmArgs a;
      a.M = M; a.H = Hn; a.U = U[n];
      a.mscale = colscale;
      a.hscale = (o->warm == CSTF_WARM_SCALED) ? nullptr : colscale + R;
      a.I = I; a.R = R; a.inv = w.inv.as<double>(); a.scal = w.scal.as<double>(); a.flag = flag;
      a.tol = o->admm.tol; a.max_iter = o->admm.max_iter; a.prox = o->admm.prox; a.variant = o->admm.variant;
      a.alpha = o->admm.alpha;
      bool fused = false;
      int iters = 0;
      if (o->update == CSTF_UPDATE_ADMM) {
        fused = admm_can_fuse_gram(R, o->admm.tol);
        a.G = fused ? Gn : nullptr;      // a7 fused into the ADMM epilogue
        double* peerH[8];
        if (peers) {                     // f4: this rank's rows go straight into every replica
          int np = 0;
          for (int r = 0; r < X->nranks; r++)
            if (r != X->rank) peerH[np++] = w.ipc_peer[r] + facoff[n] + off[n];
          a.peerH = peerH;
          a.npeer = np;
        }
        CSTF_TRY(admm_run(a, comm, st, nullptr, &iters, nullptr));
      } else {                           // f1: HALS / MU on the same M, S
        UpdArgs u;
        u.M = M; u.H = Hn; u.S = w.S.as<double>(); u.mscale = colscale; u.hscale = a.hscale;
        u.flag = flag; u.I = I; u.R = R; u.sweeps = o->admm.max_iter;
        if (o->update == CSTF_UPDATE_MU) {
          fused = R <= 32;
          u.G = fused ? Gn : nullptr;
          CSTF_TRY(mu_run(u, st));
        } else {
          CSTF_TRY(hals_run(u, st));
        }
        iters = o->admm.max_iter;
      }
      if (rep && rep->admm_iters) rep->admm_iters[t * N + n] = iters;
      tm.end(n, CSTF_PHASE_UPDATE);
      // the hot-row table of factor n follows its update (the next MTTKRPs read it);
      // distributed: from the full replica, once every rank's rows are in (below)
      if (!dist) CSTF_TRY(hot_refresh(X, n, Hn, R, st));
      // a7 (when not fused): raw Gram; a6: lambda and the normalised Gram
      if (!fused) {
        tm.begin(n, CSTF_PHASE_GRAM);
        CSTF_TRY(gram_raw(Hn, I, R, Gn, st));
        tm.end(n, CSTF_PHASE_GRAM);
      }
      if (dist && !a.peer_done) {        // every rank needs the updated factor for the next MTTKRPs
        tm.begin(n, CSTF_PHASE_COMM);
        CSTF_TRY(comm_allgather_f64(comm, Hn, fac[n], (size_t)I * R, st));
        tm.end(n, CSTF_PHASE_COMM);
      }
      // (with peer stores, the all-reduce of the Gram below is the barrier after
      // which every replica holds every rank's rows: each rank joins it only after
      // its ADMM kernel -- which ends with a system-scope fence -- has completed)
      tm.begin(n, CSTF_PHASE_NORMALIZE);
      CSTF_TRY(comm_allreduce_f64(comm, Gn, (size_t)R * R, st));
      CSTF_TRY(gram_to_lambda(Gn, R, lam + n * R, st));
      tm.end(n, CSTF_PHASE_NORMALIZE);
      if (dist) CSTF_TRY(hot_refresh(X, n, fac[n], R, st));
      if (hout && t == o->outer_iters - 1) {   // final factor n: normalised copy to the host now
        double* sn = w.stage.as<double>() + stage_off[n];
        CSTF_CUDA(cudaMemcpyAsync(sn, fac[n], (size_t)Ifull[n] * R * 8, cudaMemcpyDeviceToDevice, st));
        CSTF_TRY(scale_rows_by_cols(sn, Ifull[n], R, lam + n * R, 1, st));
        CSTF_CUDA(cudaEventRecord(w.ev_out[n], st));
        CSTF_CUDA(cudaStreamWaitEvent(w.copy, w.ev_out[n], 0));
        CSTF_CUDA(cudaMemcpyAsync(hio->out[n], sn, (size_t)Ifull[n] * R * 8, cudaMemcpyDeviceToHost, w.copy));
      }
    }
    // a8: fit of [[lambda^(N); H]]: inner product of M'(N) diag(mscale) with H_raw(N)
    tm.begin(N - 1, CSTF_PHASE_NORMALIZE);
    double* fb = w.fitbuf.as<double>();
    double* fo = sync_each ? fb : w.fits.as<double>() + 2 * t;
    CSTF_TRY(fit(X->normX2, Iloc[N - 1], R, M, fac[N - 1] + off[N - 1], colscale, lam + (N - 1) * R, G, N, fb + 4,
                 fo, flag, comm, st));
    tm.end(N - 1, CSTF_PHASE_NORMALIZE);
    if (!sync_each) {                 // fixed iteration count: no host round trip per iteration
      if (rep) rep->outer_done = t + 1;
      continue;
    }
    CSTF_CUDA(cudaMemcpyAsync(w.host_small, fb, 8, cudaMemcpyDeviceToHost, st));
    {                                 // synchronises; the flags derive from replicated / all-reduced
      cstf_status fs = check_flag(flag, st);     // values, the agreement makes that explicit
      if (dist) fs = agree(w, comm, fs, st);
      CSTF_TRY(fs);
    }
    tm.collect();
    const double f = w.host_small[0];
    if (rep) {
      if (rep->fit) rep->fit[t] = f;
      rep->outer_done = t + 1;
    }
    if (t > 0 && std::fabs(f - fit_prev) < o->fit_tol) break;
    fit_prev = f;
  }
  if (!sync_each) {                   // fits and the status flag of all iterations at once
    std::vector<double> fits((size_t)2 * o->outer_iters);
    CSTF_CUDA(cudaMemcpyAsync(fits.data(), w.fits.p, fits.size() * 8, cudaMemcpyDeviceToHost, st));
    {
      cstf_status fs = check_flag(flag, st);     // synchronises
      if (dist) fs = agree(w, comm, fs, st);
      CSTF_TRY(fs);
    }
    tm.collect();
    if (rep && rep->fit)
      for (int t = 0; t < o->outer_iters; t++) rep->fit[t] = fits[(size_t)2 * t];
  }
  // normalise the factors once (Alg. 1 l.11 applied to the final state)
  for (int n = 0; n < N; n++) {
    CSTF_TRY(scale_rows_by_cols(fac[n], Ifull[n], R, lam + n * R, 1, st));
    if (dist) CSTF_TRY(relabel_rows(fac[n], X->relabel[n].as<int32_t>(), X->dims[n], R, d_factors[n], 0, st));
  }
  if (d_lambda)
    CSTF_CUDA(cudaMemcpyAsync(d_lambda, lam + (N - 1) * R, (size_t)R * 8, cudaMemcpyDeviceToDevice, st));
  if (hio && hio->out && !hout)      // no overlap possible (fit_tol or distributed): copy at the end
    for (int n = 0; n < N; n++)
      CSTF_CUDA(cudaMemcpyAsync(hio->out[n], d_factors[n], (size_t)X->dims[n] * R * 8, cudaMemcpyDeviceToHost, st));
  CSTF_CUDA(cudaStreamSynchronize(st));
  if (hin || hout) CSTF_CUDA(cudaStreamSynchronize(w.copy));
  return CSTF_OK;
}

}  // namespace

extern "C" {

cstf_status cstf_tensor_load_coo(int nmodes, const int64_t* dims, int64_t nnz,
                                 const int32_t* const* host_idx, const double* host_vals,
                                 const cstf_comm* comm, void* stream, cstf_tensor** out) {
  if (!out) return fail(CSTF_ERR_INVALID_ARG, "out is NULL");
  *out = nullptr;
  if (nmodes < 2 || nmodes > 8) return fail(CSTF_ERR_INVALID_ARG, "nmodes must be in [2, 8]");
  if (!dims || nnz < 0) return fail(CSTF_ERR_INVALID_ARG, "dims NULL or nnz < 0");
  if (nnz >= (int64_t)1 << 32) return fail(CSTF_ERR_UNSUPPORTED, "nnz >= 2^32");
  if (nnz > 0 && (!host_idx || !host_vals)) return fail(CSTF_ERR_INVALID_ARG, "host arrays NULL");
  for (int n = 0; n < nmodes; n++) {
    if (dims[n] < 1 || dims[n] > 2147483647LL) return fail(CSTF_ERR_INVALID_ARG, "dims[n] must be in [1, 2^31-1]");
    if (nnz > 0 && !host_idx[n]) return fail(CSTF_ERR_INVALID_ARG, "host_idx[n] is NULL");
  }
  cstf_tensor* X = new cstf_tensor();
  X->N = nmodes;
  X->nranks = comm_nranks(comm);
  X->rank = comm_rank(comm);
  X->partitioned = comm != nullptr;
  for (int n = 0; n < nmodes; n++) X->dims[n] = dims[n];
  cudaGetDevice(&X->device);
  cstf_status s = build_store(X, host_idx, host_vals, nnz, S(stream));
  if (s != CSTF_OK) { delete X; return s; }
  *out = X;
  return CSTF_OK;
}

cstf_status cstf_tensor_info(const cstf_tensor* X, int* nmodes, int64_t* dims, int64_t* nnz_coalesced,
                             double* normX2, uint64_t* canonical_hash) {
  if (!X) return fail(CSTF_ERR_INVALID_ARG, "tensor is NULL");
  if (nmodes) *nmodes = X->N;
  if (dims) for (int n = 0; n < X->N; n++) dims[n] = X->dims[n];
  if (nnz_coalesced) *nnz_coalesced = X->nnz;
  if (normX2) *normX2 = X->normX2;
  if (canonical_hash) *canonical_hash = X->hash;
  return CSTF_OK;
}

cstf_status cstf_tensor_layout(const cstf_tensor* X, int mode, int64_t* nblk, int64_t* blk_rows, int* blk_mode) {
  if (!X || mode < 0 || mode >= X->N) return fail(CSTF_ERR_INVALID_ARG, "tensor is NULL or bad mode");
  const ModeStore& ms = X->mode[mode];
  if (nblk) *nblk = ms.tiled ? ms.nblk : 1;
  if (blk_rows) *blk_rows = ms.tiled ? ms.blk_rows : 0;
  if (blk_mode) *blk_mode = ms.tiled ? ms.other[ms.tslot] : -1;
  return CSTF_OK;
}

cstf_status cstf_tensor_record_bytes(const cstf_tensor* X, int mode, int* record_bytes) {
  if (!X || !record_bytes || mode < 0 || mode >= X->N) return fail(CSTF_ERR_INVALID_ARG, "tensor is NULL or bad mode");
  *record_bytes = X->mode[mode].recb;
  return CSTF_OK;
}

cstf_status cstf_tensor_export_coo(const cstf_tensor* X, int32_t* const* host_idx, double* host_vals) {
  if (!X || (X->nnz > 0 && (!host_idx || !host_vals))) return fail(CSTF_ERR_INVALID_ARG, "export arguments");
  if (X->partitioned) return fail(CSTF_ERR_UNSUPPORTED, "export of a partitioned tensor");
  return export_store(X, host_idx, host_vals);
}

void cstf_tensor_free(cstf_tensor* X) { delete X; }

cstf_status cstf_mttkrp(const cstf_tensor* X, int mode, int R, const double* const* d_factors, double* d_M,
                        void* stream) {
  if (!X || !d_factors || !d_M) return fail(CSTF_ERR_INVALID_ARG, "NULL argument");
  if (mode < 0 || mode >= X->N) return fail(CSTF_ERR_INVALID_ARG, "mode out of range");
  if (X->partitioned) return fail(CSTF_ERR_UNSUPPORTED, "cstf_mttkrp on a partitioned tensor (use cstf_factorize)");
  if (!rank_ok(R)) return fail(CSTF_ERR_UNSUPPORTED, "R must be in [1, 128]");
  for (int k = 0; k < X->N; k++)
    if (k != mode && !d_factors[k]) return fail(CSTF_ERR_INVALID_ARG, "factor pointer is NULL");
  return mttkrp(X, mode, R, d_factors, d_M, S(stream), nullptr);
}

cstf_status cstf_gram(const double* d_H, int64_t I, int R, double* d_G, const cstf_comm* comm, void* stream) {
  if ((!d_H && I > 0) || !d_G || I < 0) return fail(CSTF_ERR_INVALID_ARG, "NULL argument or I < 0");
  if (!rank_ok(R)) return fail(CSTF_ERR_UNSUPPORTED, "R must be in [1, 128]");
  return gram_normalize(const_cast<double*>(d_H), I, R, d_G, nullptr, comm, S(stream), nullptr);
}

cstf_status cstf_normalize(double* d_H, int64_t I, int R, double* d_lambda, double* d_G, const cstf_comm* comm,
                           void* stream) {
  if ((!d_H && I > 0) || !d_lambda || I < 0) return fail(CSTF_ERR_INVALID_ARG, "NULL argument or I < 0");
  if (!rank_ok(R)) return fail(CSTF_ERR_UNSUPPORTED, "R must be in [1, 128]");
  DevBuf tmp;
  double* G = d_G;
  if (!G) { CSTF_TRY(tmp.alloc((size_t)R * R * 8)); G = tmp.as<double>(); }
  CSTF_TRY(gram_normalize(d_H, I, R, G, d_lambda, comm, S(stream), nullptr));
  if (!d_G) CSTF_CUDA(cudaStreamSynchronize(S(stream)));
  return CSTF_OK;
}

cstf_status cstf_admm_update(const double* d_M, const double* d_S, double* d_H, double* d_U, int64_t I, int R,
                             const cstf_admm_opts* opts, const cstf_comm* comm, cstf_admm_stats* host_stats,
                             void* stream) {
  if (!opts || !d_S || I < 0 || (I > 0 && (!d_M || !d_H || !d_U)))
    return fail(CSTF_ERR_INVALID_ARG, "NULL argument or I < 0");
  if (!rank_ok(R)) return fail(CSTF_ERR_UNSUPPORTED, "R must be in [1, 128]");
  if (opts->max_iter < 1 || opts->tol < 0.0) return fail(CSTF_ERR_INVALID_ARG, "max_iter < 1 or tol < 0");
  if (opts->prox < CSTF_PROX_NONNEG || opts->prox > CSTF_PROX_BOX || !(opts->alpha >= 0.0) ||
      (opts->prox == CSTF_PROX_BOX && !(opts->alpha > 0.0)))
    return fail(CSTF_ERR_INVALID_ARG, "unknown prox, alpha < 0, or box bound alpha <= 0");
  cudaStream_t st = S(stream);
  DriverWs& w = dws();
  CSTF_TRY(w.inv.ensure((size_t)R * R * 8));
  CSTF_TRY(w.scal.ensure(64));
  CSTF_TRY(w.flag.ensure(64));
  int* flag = w.flag.as<int>();
  CSTF_CUDA(cudaMemsetAsync(flag, 0, 4, st));
  CSTF_TRY(chol_inverse(d_S, nullptr, 0, -1, R, opts->rho, w.inv.as<double>(), w.scal.as<double>(), flag, st));
  AdmmArgs a;
  a.M = d_M; a.H = d_H; a.U = d_U; a.hscale = nullptr; a.I = I; a.R = R;
  a.inv = w.inv.as<double>(); a.scal = w.scal.as<double>(); a.flag = flag;
  a.tol = opts->tol; a.max_iter = opts->max_iter; a.prox = opts->prox; a.variant = opts->variant;
  a.alpha = opts->alpha;
  cstf_admm_stats stats;
  CSTF_TRY(admm_run(a, comm, st, &stats, nullptr, nullptr));
  CSTF_TRY(check_flag(flag, st));
  if (host_stats) *host_stats = stats;
  return CSTF_OK;
}

static cstf_status run_update(int kind, const double* d_M, const double* d_S, double* d_H, int64_t I, int R,
                              int sweeps, void* stream) {
  if (!d_S || I < 0 || (I > 0 && (!d_M || !d_H))) return fail(CSTF_ERR_INVALID_ARG, "NULL argument or I < 0");
  if (!rank_ok(R)) return fail(CSTF_ERR_UNSUPPORTED, "R must be in [1, 128]");
  if (sweeps < 1) return fail(CSTF_ERR_INVALID_ARG, "sweeps < 1");
  DriverWs& w = dws();
  CSTF_TRY(w.flag.ensure(64));
  CSTF_CUDA(cudaMemsetAsync(w.flag.p, 0, 4, S(stream)));
  UpdArgs u;
  u.M = d_M; u.H = d_H; u.S = d_S; u.flag = w.flag.as<int>(); u.I = I; u.R = R; u.sweeps = sweeps;
  return kind == CSTF_UPDATE_MU ? mu_run(u, S(stream)) : hals_run(u, S(stream));
}

cstf_status cstf_hals_update(const double* d_M, const double* d_S, double* d_H, int64_t I, int R, int sweeps,
                             void* stream) {
  return run_update(CSTF_UPDATE_HALS, d_M, d_S, d_H, I, R, sweeps, stream);
}

cstf_status cstf_mu_update(const double* d_M, const double* d_S, double* d_H, int64_t I, int R, int sweeps,
                           void* stream) {
  return run_update(CSTF_UPDATE_MU, d_M, d_S, d_H, I, R, sweeps, stream);
}

cstf_status cstf_release_workspace(void) {
  CSTF_CUDA(cudaDeviceSynchronize());       // no launch of this thread may still use them
  DriverWs& w = dws();
  for (int r = 0; r < 8; r++)
    if (w.ipc_peer[r]) { cudaIpcCloseMemHandle(w.ipc_peer[r]); w.ipc_peer[r] = nullptr; }
  w.ipc_state = 0;
  for (DevBuf* b : {&w.grams, &w.lam, &w.inv, &w.scal, &w.flag, &w.fitbuf, &w.fits, &w.M, &w.U, &w.hostfac, &w.S,
                    &w.stage, &w.facall, &w.xchg, &w.agreebuf})
    b->release();
  for (int n = 0; n < 8; n++) w.Fi[n].release();
  w.facall_gen++;
  release_mttkrp_ws();
  release_admm_ws();
  release_dense_ws();
  return CSTF_OK;
}

cstf_status cstf_factorize(const cstf_tensor* X, const cstf_opts* opts, const cstf_comm* comm,
                           double* const* d_factors, double* d_lambda, cstf_report* report, void* stream) {
  if (!X || !opts || !d_factors) return fail(CSTF_ERR_INVALID_ARG, "NULL argument");
  return factorize_impl(X, opts, comm, d_factors, d_lambda, report, S(stream));
}

cstf_status cstf_factorize_host(const cstf_tensor* X, const cstf_opts* opts, const cstf_comm* comm,
                                double* const* host_factors, double* host_lambda, cstf_report* report,
                                void* stream) {
  if (!X || !opts || !host_factors) return fail(CSTF_ERR_INVALID_ARG, "NULL argument");
  if (!rank_ok(opts->R)) return fail(CSTF_ERR_UNSUPPORTED, "R must be in [1, 128]");
  cudaStream_t st = S(stream);
  DriverWs& w = dws();
  const int N = X->N, R = opts->R;
  int64_t tot = 0;
  for (int n = 0; n < N; n++) tot += X->dims[n] * R;
  CSTF_TRY(w.hostfac.ensure((size_t)(tot + R) * 8));
  std::vector<double*> d(N);
  int64_t off = 0;
  const bool dist = X->partitioned;
  for (int n = 0; n < N; n++) {
    if (!host_factors[n]) return fail(CSTF_ERR_INVALID_ARG, "host factor pointer is NULL");
    d[n] = w.hostfac.as<double>() + off;
    if (dist)                        // (the partitioned path relabels from device copies first)
      CSTF_CUDA(cudaMemcpyAsync(d[n], host_factors[n], (size_t)X->dims[n] * R * 8, cudaMemcpyHostToDevice, st));
    off += X->dims[n] * R;
  }
  double* d_lam = w.hostfac.as<double>() + off;
  HostIO io;
  io.in = dist ? nullptr : host_factors;
  io.out = host_factors;
  const cstf_status fs = factorize_impl(X, opts, comm, d.data(), d_lam, report, st, &io);
  if (fs != CSTF_OK) {               // no copy may touch the caller's buffers after the return
    cudaStreamSynchronize(st);
    cudaStreamSynchronize(w.copy);
    return fs;
  }
  if (host_lambda) CSTF_CUDA(cudaMemcpyAsync(host_lambda, d_lam, (size_t)R * 8, cudaMemcpyDeviceToHost, st));
  CSTF_CUDA(cudaStreamSynchronize(st));
  return CSTF_OK;
}

}  // extern "C"
