// Internal declarations of libcstf (host C++ / CUDA, sm_100a).  Not part of the ABI.
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <string>
#include <vector>

#include "../../include/cstf.h"

namespace cstf {

// ---------------------------------------------------------------- errors
void set_error(const std::string& msg);
cstf_status fail(cstf_status s, const std::string& msg);
cstf_status cuda_fail(cudaError_t e, const char* what);

#define CSTF_CUDA(call)                                          \
  do {                                                           \
    cudaError_t e_ = (call);                                     \
    if (e_ != cudaSuccess) return ::cstf::cuda_fail(e_, #call);  \
  } while (0)
#define CSTF_TRY(call)                         \
  do {                                         \
    cstf_status s_ = (call);                   \
    if (s_ != CSTF_OK) return s_;              \
  } while (0)
// after a kernel launch
#define CSTF_LAUNCHED() \
  do { ::cstf::count_launch(); CSTF_CUDA(cudaGetLastError()); } while (0)

void count_launch(int n = 1);

// ---------------------------------------------------------------- device info
struct DeviceInfo {
  int device = -1;
  int sms = 0;
  size_t l2 = 0;
  int max_smem_optin = 0;
};
const DeviceInfo& device_info();

// ---------------------------------------------------------------- buffers
// Owned device allocation (cudaMalloc / cudaFree).
struct DevBuf {
  void* p = nullptr;
  size_t bytes = 0;
  DevBuf() = default;
  DevBuf(const DevBuf&) = delete;
  DevBuf& operator=(const DevBuf&) = delete;
  DevBuf(DevBuf&& o) noexcept : p(o.p), bytes(o.bytes) { o.p = nullptr; o.bytes = 0; }
  DevBuf& operator=(DevBuf&& o) noexcept {
    if (this != &o) { release(); p = o.p; bytes = o.bytes; o.p = nullptr; o.bytes = 0; }
    return *this;
  }
  ~DevBuf() { release(); }
  void release();
  cstf_status alloc(size_t n);          // exact (re)allocation, contents undefined
  cstf_status ensure(size_t n);         // grow-only
  template <class T> T* as() const { return static_cast<T*>(p); }
};

// ---------------------------------------------------------------- comm
struct Comm {
  int nranks = 1;
  int rank = 0;
  void* nccl = nullptr;  // ncclComm_t
  cstf_host_allreduce_fn host_allreduce = nullptr;   // host-callback transport
  cstf_host_allgather_fn host_allgather = nullptr;
  void* user = nullptr;
  void* loop = nullptr;  // cstf_comm_loopback member (owned)
};
cstf_status comm_allreduce_f64(const cstf_comm* c, double* d_buf, size_t count, cudaStream_t st);
cstf_status comm_allgather_f64(const cstf_comm* c, const double* d_send, double* d_recv,
                               size_t count_per_rank, cudaStream_t st);
int comm_nranks(const cstf_comm* c);
int comm_rank(const cstf_comm* c);

// ---------------------------------------------------------------- tensor store
// Mode-n copy of the nonzeros: sorted by i_n, then by the other modes in
// increasing length order (so fibers of the shortest other mode are contiguous).
// Array-of-structs records of `recb` bytes: int32 index of other[q] at byte 4q,
// the FP64 value in the last 8 bytes.
//
// k-blocked copies: when the output mode is short and the
// longest other mode is long, the nonzeros are ordered by (kb = i_t / kTileRows,
// i_n, ...), t = other[N-2].  Rows are then "virtual rows" v = kb * I + i_n and
// rowptr has nblk * I + 1 entries; MTTKRP writes one partial row per virtual row
// and sums the partials over kb in fixed order.  The factor rows of block kb are
// staged in shared memory by the CTA that processes them.
constexpr int kTileRows = 256;        // SMEM-slab blocks (opt-in CSTF_KBLOCK=1)
constexpr int64_t kL2Rows = 100000;     // L2 blocks: 25.6 / 51.2 MB of factor rows at R = 32 / 64
struct ModeStore {
  int64_t I = 0;            // rows of this mode (local rows when distributed)
  int64_t nnz = 0;          // nonzeros in this copy
  DevBuf rowptr;            // int64[Ivirt+1]
  DevBuf rec;               // nnz records
  int recb = 16;            // record bytes: round_up(4 (N-1) + 8, 16)
  int other[7];             // mode id of record slot q (slot 0 = shortest other mode)
  // k-blocking
  bool tiled = false;
  bool slab = false;        // blocks of kTileRows staged in SMEM (else L2-sized blocks)
  int64_t blk_rows = 0;     // rows of the blocked mode per block
  int tslot = 0;            // record slot of the blocked mode
  int64_t nblk = 1;         // blocks of the tiled mode
  int64_t Ivirt = 0;        // rows of rowptr (= I when not tiled)
  // cached work split of a tiled copy: warp-chunk starts and the block of each CTA chunk
  mutable DevBuf wstart;    // int64[nwchunks+1]
  mutable DevBuf ckb;       // int32[nctachunks]
  mutable int64_t nwchunks = 0, nctachunks = 0;
  // cached chunk boundaries of the MTTKRP work split (depend only on the store)
  mutable DevBuf clb, ccont;
  mutable int64_t cchunk = -1, cnchunks = 0;
  mutable std::vector<int64_t> kp;   // L2-blocked copies: first nonzero of each block (host, cached)
  // hot-row tables: bit q set = the records of slot q name hot rows of factor other[q]
  // by (0x80000000 | hot slot)
  int hotmask = 0;
  // Packed 16-byte records (round 2): when the row indices of
  // the N-1 = 3 gathered slots fit one 64-bit word, record = {uint64 key, f64 x} with
  // slot q at bits [pk_sh[q], pk_sh[q] + width) of key: the row, or pk_hot[q] | hot slot
  // (pk_hot[q] = the field's top bit, 0 for slots without hot rows).  In an L2-blocked
  // copy the blocked slot stores its row within the block (pk_rel = tslot; the block is
  // the one of the virtual row).  CSTF_PACK=0 keeps the 32-byte records.
  bool pk = false;
  int pk_rel = -1;          // L2-blocked packed copy: slot tslot holds the row within its block
  int pk_sh[7] = {0};
  uint32_t pk_mask[7] = {0};
  uint32_t pk_hot[7] = {0};
};
inline int record_bytes(int N) { return ((4 * (N - 1) + 8) + 15) / 16 * 16; }

}  // namespace cstf

struct cstf_comm {
  cstf::Comm c;
};

struct cstf_tensor {
  int N = 0;
  int64_t dims[8] = {0};
  int64_t nnz = 0;          // coalesced (local share when distributed)
  double normX2 = 0.0;
  uint64_t hash = 0;
  int device = -1;
  cstf::ModeStore mode[8];
  // distributed layout (nranks > 1): rows of mode n are dealt to ranks
  // (cstf_partition_rows); internal label of row i = owner(i) * B_n + local(i),
  // so every rank's rows are one contiguous slice [rank*B_n, (rank+1)*B_n) of the
  // internal (relabelled, zero-padded) factor of P*B_n rows.
  int nranks = 1, rank = 0;
  bool partitioned = false;           // loaded with a communicator (any size): row-partitioned layout
  int64_t rows_per_rank[8] = {0};     // B_n
  cstf::DevBuf relabel[8];            // int32[dims[n]]: internal label of original row
  // Hot-row tables (single GPU, factors much larger than L2): the rows of factor k
  // with the most nonzeros get hot slots hot_off[k] .. hot_off[k] + hot_cnt[k] - 1
  // of one table (hot_total rows x R), refreshed from the factor and read by MTTKRP
  // under a persisting L2 access window, so the L2 keeps exactly the rows most
  // gathers hit.  hot_rows[hot slot] = factor row.
  int64_t hot_cnt[8] = {0}, hot_off[8] = {0}, hot_total = 0;
  cstf::DevBuf hot_rows;              // int32[hot_total]
  mutable cstf::DevBuf hot_tab;       // hot_total x hot_R doubles (allocated on first use)
  mutable int hot_R = 0;
};

namespace cstf {

// ---------------------------------------------------------------- kernels (launchers)
// store.cu
cstf_status build_store(cstf_tensor* X, const int32_t* const* host_idx, const double* host_vals,
                        int64_t nnz_in, cudaStream_t st);
cstf_status export_store(const cstf_tensor* X, int32_t* const* host_idx, double* host_vals);

// mttkrp.cu
// hot_fresh: the hot-row tables already hold the current rows of every factor the
// copy gathers (factorize refreshes them after each update); else they are refreshed
// from d_factors first.
cstf_status mttkrp(const cstf_tensor* X, int mode, int R, const double* const* d_factors,
                   double* d_M, cudaStream_t st, int64_t* launches, bool hot_fresh = false);
// copy the hot rows of factor k (d_F, I_k x R) into X's hot table (allocated for R)
cstf_status hot_refresh(const cstf_tensor* X, int k, const double* d_F, int R, cudaStream_t st);
// persisting-L2 set-aside for the hot tables: set (saving the caller's) / restore + reset
struct L2Persist {
  size_t saved = 0;
  bool active = false;
};
cstf_status hot_persist_begin(const cstf_tensor* X, L2Persist& p);
void hot_persist_end(L2Persist& p);

// dense.cu
// G (R x R) = H^T H; if lam != nullptr also normalises: lam_r = sqrt(G_rr), H /= lam (in place),
// G <- D^-1 G D^-1.  comm: all-reduce the raw Gram.
cstf_status gram_normalize(double* d_H, int64_t I, int R, double* d_G, double* d_lam,
                           const cstf_comm* comm, cudaStream_t st, int64_t* launches);
// pieces of gram_normalize (no comm): raw Gram, then lam / G scaling / H /= lam
cstf_status gram_raw(const double* d_H, int64_t I, int R, double* d_G, cudaStream_t st);
cstf_status normalize_from_gram(double* d_H, int64_t I, int R, double* d_G, double* d_lam,
                                cudaStream_t st);
cstf_status fill(double* d, int64_t n, double v, cudaStream_t st);
// One CTA: S = Hadamard of the Grams except `skip` (or copy of d_S when grams == nullptr),
// rho, Cholesky of S + rho I, Inv = (S + rho I)^-1.  Writes d_inv (R x R), d_scal[0] = rho,
// d_flag |= 1 on NOT_SPD.
// With d_lam (N x R, lazy normalisation) also writes d_colscale[0..R) =
// prod_{k != skip} 1/lambda_k (0 where lambda_k = 0) and d_colscale[R..2R) = 1/lambda_skip.
cstf_status chol_inverse(const double* d_S, const double* d_grams, int N, int skip, int R,
                         double rho_in, double* d_inv, double* d_scal, int* d_flag,
                         cudaStream_t st, const double* d_lam = nullptr, double* d_colscale = nullptr,
                         double* d_S_out = nullptr);
// lambda_r = sqrt(G_rr); G <- D^-1 G D^-1 (H untouched)
cstf_status gram_to_lambda(double* d_G, int R, double* d_lam, cudaStream_t st);
// fit (D12): writes d_out[0] = fit.  inner = sum_i sum_r M_ir H_ir colw_r, xhat = lam^T (*G) lam.
// (lazy normalisation: M = MTTKRP of the raw factors, H = raw last factor, colw = its mscale)
cstf_status fit(double normX2, int64_t I, int R, const double* d_M, const double* d_H,
                const double* d_colw, const double* d_lam, const double* d_grams, int N,
                double* d_part /* >= 256 */, double* d_out /* [2] */, int* d_flag,
                const cstf_comm* comm, cudaStream_t st);
cstf_status scale_rows_by_cols(double* d_H, int64_t I, int R, const double* d_lam, int divide,
                               cudaStream_t st);

// admm.cu
struct AdmmArgs {
  const double* M;
  double* H;
  double* U;
  const double* hscale;  // optional per-column scale of the incoming H
  const double* mscale = nullptr;  // optional per-column scale of M (lazy normalisation)
  double* G = nullptr;   // optional: raw Gram H^T H of the result (fused epilogue)
  int64_t I;
  int R;
  const double* inv;     // device R x R
  const double* scal;    // device: [0] = rho
  int* flag;             // device status flags
  double tol;
  int max_iter;
  int prox;
  int variant;
  double alpha = 0.0;    // L1 weight (prox 2/3)
  double* const* peerH = nullptr;  // fused all-gather: this rank's rows in each peer replica
  int npeer = 0;
  mutable bool peer_done = false;  // out: the rows were stored into the peers
};
cstf_status admm_run(const AdmmArgs& a, const cstf_comm* comm, cudaStream_t st,
                     cstf_admm_stats* stats, int* iters_out, int64_t* launches);
bool admm_can_fuse_gram(int R, double tol);
// G = H^T H on the DMMA path for R <= 64 (returns false if not applicable; *status = launch status)
bool gram_dmma(const double* d_H, int64_t I, int R, double* d_G, cudaStream_t st, cstf_status* status);

// f1 update schemes (HALS / MU), same row-wise shape as ADMM
struct UpdArgs {
  const double* M;
  double* H;
  const double* S;        // R x R Hadamard of Grams
  const double* mscale = nullptr;
  const double* hscale = nullptr;
  const double* scal = nullptr;   // unused by HALS/MU (rho slot)
  const int* flag;
  double* G = nullptr;    // MU: fused raw Gram of the result (R <= 32)
  int64_t I;
  int R;
  int sweeps;
};
cstf_status hals_run(const UpdArgs& a, cudaStream_t st);

// cached per-thread, per-device workspaces (cstf_release_workspace)
void release_mttkrp_ws();
void release_admm_ws();
void release_dense_ws();
cstf_status mu_run(const UpdArgs& a, cudaStream_t st);

}  // namespace cstf
