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
#include <cstdlib>
#include <vector>

#include "internal.h"

namespace cstf {
namespace {

constexpr int kWarps = 8;  // per CTA

// Resident CTAs per SM of the fast kernel (its register budget) by average nonzeros
// per row: < 16 -> 4 (64 registers: row flushes dominate, latency hiding needs
// warps), < 64 -> 3 for R = 32 / 64 (80 registers; Delicious mode 2, 56 per row:
// 10.81 -> 10.0 ms), else 2 (long rows).  Virtual rows of L2-blocked copies (`tiled`)
// keep 4 below 64 (Amazon, ~20 per virtual row: 531 -> 592 ms with 3).
// Hot-row copies at R = 32 (factors streamed from HBM) trade warps for gathers in
// flight per warp (mttkrp_unr): short rows 3 CTAs with 2 steps of row loads issued
// together, medium rows 2 CTAs with 4 steps (bench path, Delicious modes 1 / 2:
// 11.84 -> 11.26 ms, 9.90 -> 9.44 ms; tools/bench_variants.sh,
// profiles/r02_mttkrp_unroll_variants.txt).
// CSTF_MTTKRP_MINB=2/3/4 and CSTF_MTTKRP_UNR=1..4 force (experiments).
int mttkrp_minb(int64_t nnz, int64_t rows, int R, bool tiled, bool hot = false, int nother = 3) {
  if (const char* e = getenv("CSTF_MTTKRP_MINB")) {
    const int v = atoi(e);
    if (v == 2 || v == 4 || (v == 3 && (R == 32 || R == 64))) return v;
  }
  if (hot && R == 32 && !tiled && nother <= 4 && nnz < 64 * rows) return nnz < 16 * rows ? 3 : 2;
  if (nnz < 16 * rows) return 4;
  if (nnz < 64 * rows) return (!tiled && (R == 32 || R == 64)) ? 3 : 4;
  return 2;
}

// Hot-row copies of 4-mode tensors at R = 32 with >= 16 nonzeros per row (not L2-blocked):
// 8-lane groups with 2 steps of row loads in flight (Delicious mode 0 9.19 -> 8.99 ms,
// mode 2 9.36 -> 9.12 ms; short rows stay on 16-lane groups: mode 1 11.26 -> 11.56 ms with
// 8; profiles/r02_mttkrp_g8_hot_probe.txt).  The group width depends on the row class only,
// so forced unroll depths (CSTF_MTTKRP_UNR) keep the accumulation order.
bool mttkrp_hot_g8(int64_t nnz, int64_t rows, int R, bool tiled, bool hot, int nother) {
  if (!(hot && R == 32 && !tiled && nother == 3 && nnz >= 16 * rows)) return false;
  const char* ge = getenv("CSTF_MTTKRP_G");      // CSTF_MTTKRP_G=0: 16-lane groups everywhere (tests)
  return !(ge && atoi(ge) == 0);
}

// Steps of row gathers issued before the first product (hot-row copies, R = 32; 1 elsewhere)
int mttkrp_unr(int64_t nnz, int64_t rows, int R, bool tiled, bool hot, int nother = 3) {
  if (!hot || R != 32 || nother > 4) return 1;
  if (const char* e = getenv("CSTF_MTTKRP_UNR")) {
    const int v = atoi(e);
    if (v >= 1 && v <= 4) return v;
  }
  if (mttkrp_hot_g8(nnz, rows, R, tiled, hot, nother)) return 2;
  if (tiled || nnz >= 64 * rows) return 1;
  return nnz < 16 * rows ? 2 : 4;
}

struct MArgs {
  const int64_t* rowptr;
  const char* rec;
  const double* F[7];   // factor of record slot q
  int64_t I, nnz, chunk, nchunks;   // I: end row (absolute); nnz: nonzeros of this launch
  int64_t pbase, rbase;             // first nonzero / first (virtual) row of this launch; a.M row 0 = rbase
  int64_t cbase;                    // absolute index of chunk 0 (chunk c = [(cbase + c) chunk, ...) clipped)
  int R, recb, nother;
  const int64_t* lb;    // [nchunks+1] first row with rowptr >= start of chunk c (lb[nchunks] = I)
  const int32_t* cont;  // [nchunks] row continuing into chunk c from an earlier chunk, or -1
  const int64_t* wstart;  // [nchunks+1] explicit chunk starts (k-blocked copies) or null
  const int32_t* ckb;     // [nchunks/8] block of each CTA chunk (k-blocked copies)
  int64_t It;             // rows of the k-blocked mode's factor (slot nother-1)
  int64_t It_blk;         // rows of the L2-blocked factor (slot tslot)
  double* M;            // output rows (virtual rows when k-blocked)
  double* carry;        // [nchunks][R]
  unsigned long long* queue;  // dynamic chunk counter (L2-blocked copies) or null = static grid stride
  const double* HF[7];  // hot-row table of the factor of slot q (records 0x80000000 | hot slot), or null
  int l2blocked;        // launch over an L2-blocked copy (rows are virtual rows)
  int pk;               // packed 16-byte records (ModeStore::pk): slot q = (key >> pk_sh[q]) & pk_mask[q]
  int pk_rel;           // L2-blocked packed copy: slot stored relative to its block (-1: none)
  uint32_t pk_blk;      //   rows per block of that slot
  int64_t Iout;         //   output rows per block (virtual row v lies in block v / Iout)
  int pk_sh[3];
  uint32_t pk_mask[3], pk_hot[3];
};

// Field of record slot q of a packed record (key = words w0, w1): the row, or the hot
// flag pk_hot[q] | hot slot
__device__ __forceinline__ unsigned pk_field(const MArgs& a, int q, unsigned w0, unsigned w1) {
  return q == 0 ? (w0 & a.pk_mask[0])
                : (unsigned)((((unsigned long long)w1 << 32) | w0) >> a.pk_sh[q]) & a.pk_mask[q];
}

// Row source and row of slot q: the hot-row table for a hot slot, else the factor.  Both
// record kinds resolve by selects (no branch, so the gathers of a step issue together).
template <bool PK, bool HOT>
__device__ __forceinline__ void slot_row(const MArgs& a, int q, const unsigned* w, const char* fb, const char* hfb,
                                         const char*& base, unsigned& j) {
  if constexpr (PK) {
    const unsigned f = pk_field(a, q, w[0], w[1]);
    if constexpr (HOT) {
      const unsigned hb = f & a.pk_hot[q];
      j = f ^ hb;
      base = hb ? hfb : fb;
    } else {
      j = f;
      base = fb;
    }
  } else {
    j = w[q];
    base = fb;
    if constexpr (HOT) {            // hot row: its copy in the persisting hot-row table
      if ((int)j < 0) { base = hfb; j &= 0x7fffffffu; }
    }
  }
}

// Chunks sit on the absolute grid of multiples of `chunk`, clipped to the launch's
// nonzero range: a launch over a batch of L2 blocks splits every row exactly where
// one launch over all blocks would (same arithmetic, bit for bit).
__device__ __forceinline__ int64_t chunk_begin(const MArgs& a, int64_t c) {
  return a.wstart ? a.wstart[c] : max(a.pbase, (a.cbase + c) * a.chunk);
}
__device__ __forceinline__ int64_t chunk_end(const MArgs& a, int64_t c) {
  return a.wstart ? a.wstart[c + 1] : min((a.cbase + c + 1) * a.chunk, a.pbase + a.nnz);
}

// Chunk c covers nonzeros [pbase + c chunk, ...) of rows [rbase, rend) (absolute
// row and nonzero positions; a launch over a batch of L2 blocks uses a sub-range).
__global__ void k_chunk_bounds(const int64_t* __restrict__ rowptr, int64_t rbase, int64_t rend, int64_t pbase,
                               int64_t pend, int64_t chunk, int64_t cbase, int64_t nchunks,
                               const int64_t* __restrict__ wstart, int64_t* __restrict__ lb,
                               int32_t* __restrict__ cont) {
  for (int64_t c = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; c <= nchunks;
       c += (int64_t)gridDim.x * blockDim.x) {
    if (c == nchunks) { lb[c] = rend; continue; }
    const int64_t p0 = wstart ? wstart[c] : max(pbase, (cbase + c) * chunk);
    int64_t lo = rbase, hi = rend;   // lower_bound: first row r with rowptr[r] >= p0
    while (lo < hi) {
      const int64_t mid = (lo + hi) >> 1;
      if (rowptr[mid] < p0) lo = mid + 1; else hi = mid;
    }
    lb[c] = lo;
    int32_t ct = -1;                 // the row containing p0 started before p0
    if (p0 < pend && lo > rbase && (lo == rend || rowptr[lo] > p0)) ct = (int32_t)(lo - 1);
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
// One warp processes chunk c.  Fb[q] = lane's byte offset into the row source of
// slot q (a factor in global memory, or the shared-memory slab of a k-blocked
// copy, already shifted by the slab's first row).
template <int NOTHER, int R, int RECB, int GL = 0, bool HOT = false, int UNR = 1, bool REL = false>
__device__ __forceinline__ void process_chunk(const MArgs& a, int64_t c, const char* const* Fb, int4* srec,
                                              const char* const* HFb = nullptr) {
  constexpr int RV = R / 2;                    // double2 per row
  constexpr int G = GL ? GL : (RV < 32 ? RV : 32);   // lanes per group
  constexpr int VPL = RV / G;                  // double2 per lane
  constexpr int P = 32 / G;                    // nonzeros per warp step
  constexpr unsigned ROWB = R * 8;
  constexpr int NW = RECB / 4;                 // 32-bit words per record
  constexpr bool PK = RECB == 16 && NOTHER >= 3;   // packed records (3 slots in one 64-bit key)
  const int lane = threadIdx.x & 31;
  const int sg = lane / G, gl = lane % G;
  {
    const int64_t p0 = chunk_begin(a, c);
    const int64_t p1 = chunk_end(a, c);
    const int32_t ct = a.cont[c];
    int64_t row = ct >= 0 ? (int64_t)ct : a.lb[c];
    const int64_t row_end = (c == a.nchunks - 1) ? a.I : a.lb[c + 1];
    double2 acc[VPL];
#pragma unroll
    for (int s = 0; s < VPL; s++) acc[s] = make_double2(0.0, 0.0);
    int64_t seg_end = (row < row_end) ? min(a.rowptr[row + 1], p1) : p1;
    // REL (packed L2-blocked copy): the blocked slot's field is the row within the block of
    // the current virtual row; kbrow = that block's first row, advanced at block changes
    uint32_t kbrow = 0;
    int64_t kb_next = 0;
    if constexpr (REL) {
      const int64_t kb = row / a.Iout;
      kbrow = (uint32_t)kb * a.pk_blk;
      kb_next = (kb + 1) * a.Iout;
    }

    auto flush = [&](int64_t r) {
#pragma unroll
      for (int off = 16; off >= G; off >>= 1)
#pragma unroll
        for (int s = 0; s < VPL; s++) {
          acc[s].x += __shfl_xor_sync(0xffffffffu, acc[s].x, off);
          acc[s].y += __shfl_xor_sync(0xffffffffu, acc[s].y, off);
        }
      if (sg == 0) {
        double* dst = (ct >= 0 && r == (int64_t)ct) ? a.carry + c * (int64_t)R : a.M + (r - a.rbase) * (int64_t)R;
#pragma unroll
        for (int s = 0; s < VPL; s++) reinterpret_cast<double2*>(dst)[gl + s * G] = acc[s];
      }
#pragma unroll
      for (int s = 0; s < VPL; s++) acc[s] = make_double2(0.0, 0.0);
    };

    // Records arrive 32 at a time: one coalesced 16-byte load per lane, issued
    // one batch ahead (register double buffer), published through a per-warp
    // shared buffer; each group then reads its record with one 16-byte LDS.
    constexpr int NV = RECB / 16;                // int4 per record
    int4* sr = srec + (threadIdx.x >> 5) * 32 * NV;
    int4 nxt[NV];
#pragma unroll
    for (int k = 0; k < NV; k++)
      nxt[k] = (p0 + lane < p1) ? __ldcs(reinterpret_cast<const int4*>(a.rec + (p0 + lane) * RECB) + k)
                                : make_int4(0, 0, 0, 0);
    for (int64_t pb = p0; pb < p1; pb += 32) {
      const int nb = (int)min((int64_t)32, p1 - pb);
      __syncwarp();
#pragma unroll
      for (int k = 0; k < NV; k++) sr[lane * NV + k] = nxt[k];
      __syncwarp();
#pragma unroll
      for (int k = 0; k < NV; k++)
        nxt[k] = (pb + 32 + lane < p1) ? __ldcs(reinterpret_cast<const int4*>(a.rec + (pb + 32 + lane) * RECB) + k)
                                       : make_int4(0, 0, 0, 0);
      int t = 0;
      while (t < nb) {
        const int64_t p = pb + t;
        if (p >= seg_end) {
          flush(row);
          row++;
          seg_end = min(a.rowptr[row + 1], p1);
          if constexpr (REL) {
            if (row >= kb_next) { kbrow += a.pk_blk; kb_next += a.Iout; }
          }
          continue;
        }
        const int run = (int)min((int64_t)(nb - t), seg_end - p);
        if constexpr (UNR > 1) {
          // UNR steps per iteration, every row load of all of them issued before the
          // first product: UNR x NOTHER gathers in flight per lane instead of NOTHER
          for (int done = 0; done < run; done += UNR * P) {
            double2 xs[UNR][NOTHER][VPL];
            double vv[UNR];
#pragma unroll
            for (int u = 0; u < UNR; u++) {
              const int d = done + u * P;
              const bool ok = (d + sg) < run;
              const int src = ok ? t + d + sg : t + done;
              unsigned w[NW];
#pragma unroll
              for (int k = 0; k < NV; k++) {
                const int4 x = sr[src * NV + k];
                w[4 * k] = x.x; w[4 * k + 1] = x.y; w[4 * k + 2] = x.z; w[4 * k + 3] = x.w;
              }
              vv[u] = ok ? __hiloint2double((int)w[NW - 1], (int)w[NW - 2]) : 0.0;
#pragma unroll
              for (int qq = 0; qq < NOTHER; qq++) {
                const char* base;
                unsigned j;
                slot_row<PK, HOT>(a, qq, w, Fb[qq], HOT ? HFb[qq] : nullptr, base, j);
                if constexpr (REL) j += (qq == a.pk_rel) ? kbrow : 0u;
                const double2* rp = row_addr<ROWB>(base, j);
#pragma unroll
                for (int s = 0; s < VPL; s++) xs[u][qq][s] = rp[s * G];
              }
            }
#pragma unroll
            for (int u = 0; u < UNR; u++)
#pragma unroll
              for (int s = 0; s < VPL; s++) {
                double2 f = xs[u][0][s];
#pragma unroll
                for (int qq = 1; qq < NOTHER; qq++) { f.x *= xs[u][qq][s].x; f.y *= xs[u][qq][s].y; }
                acc[s].x = fma(vv[u], f.x, acc[s].x);
                acc[s].y = fma(vv[u], f.y, acc[s].y);
              }
          }
          t += run;
          continue;
        }
#pragma unroll 4
        for (int done = 0; done < run; done += P) {
          const bool ok = (done + sg) < run;
          const int src = ok ? t + done + sg : t + done;      // a valid slot of this batch
          unsigned w[NW];
#pragma unroll
          for (int k = 0; k < NV; k++) {
            const int4 x = sr[src * NV + k];
            w[4 * k] = x.x; w[4 * k + 1] = x.y; w[4 * k + 2] = x.z; w[4 * k + 3] = x.w;
          }
          const double v = ok ? __hiloint2double((int)w[NW - 1], (int)w[NW - 2]) : 0.0;   // idle group adds 0
          double2 f[VPL];
#pragma unroll
          for (int qq = 0; qq < NOTHER; qq++) {
            const char* base;
            unsigned j;
            slot_row<PK, HOT>(a, qq, w, Fb[qq], HOT ? HFb[qq] : nullptr, base, j);
                if constexpr (REL) j += (qq == a.pk_rel) ? kbrow : 0u;
            const double2* rp = row_addr<ROWB>(base, j);
#pragma unroll
            for (int s = 0; s < VPL; s++) {
              const double2 x = rp[s * G];     // global (read-only) or shared slab
              if (qq == 0) f[s] = x;
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

// MINB: CTAs per SM the register budget targets (2 for long rows, 4 for short ones)
template <int NOTHER, int R, int RECB, int MINB, int GL = 0, bool HOT = false, int UNR = 1, bool REL = false>
__global__ void __launch_bounds__(kWarps * 32, MINB) k_mttkrp_fast(MArgs a) {
  constexpr int G = GL ? GL : ((R / 2) < 32 ? (R / 2) : 32);
  const int gl = (threadIdx.x & 31) % G;
  const char* Fb[NOTHER];
  const char* HFb[HOT ? NOTHER : 1];
#pragma unroll
  for (int q = 0; q < NOTHER; q++) Fb[q] = reinterpret_cast<const char*>(a.F[q]) + gl * 16;
  if constexpr (HOT) {
#pragma unroll
    for (int q = 0; q < NOTHER; q++) HFb[q] = reinterpret_cast<const char*>(a.HF[q] ? a.HF[q] : a.F[q]) + gl * 16;
  }
  const int64_t warp0 = blockIdx.x * (int64_t)kWarps + (threadIdx.x >> 5);
  const int64_t nwarps = (int64_t)gridDim.x * kWarps;
  __shared__ int4 srec[kWarps * 32 * (RECB / 16)];
  if (a.queue) {
    // L2-blocked copies: warps take chunks in global order from a counter, so the
    // nonzeros in flight span a narrow range of the blocked factor's rows (its
    // L2-resident slab) instead of grid-stride windows spread over the tensor.
    // Which warp runs a chunk does not change its arithmetic (deterministic).
    for (;;) {
      unsigned long long c = 0;
      if ((threadIdx.x & 31) == 0) c = atomicAdd(a.queue, 1ULL);
      c = __shfl_sync(0xffffffffu, c, 0);
      if ((int64_t)c >= a.nchunks) break;
      process_chunk<NOTHER, R, RECB, GL, HOT, UNR, REL>(a, (int64_t)c, Fb, srec, HFb);
    }
    return;
  }
  for (int64_t c = warp0; c < a.nchunks; c += nwarps) process_chunk<NOTHER, R, RECB, GL, HOT, UNR, REL>(a, c, Fb, srec, HFb);
}

// k-blocked copy: CTA chunk b (8 warp chunks) lies in block kb = ckb[b]; the
// block's kTileRows rows of the last slot's factor are staged in shared memory
// (coalesced 16-byte copies), the other slots gather from global memory.
template <int NOTHER, int R, int RECB>
__global__ void __launch_bounds__(kWarps * 32, 2) k_mttkrp_tiled(MArgs a) {
  extern __shared__ double2 slab[];            // [kTileRows][R/2]
  __shared__ int4 srec[kWarps * 32 * (RECB / 16)];
  constexpr int G = (R / 2) < 32 ? (R / 2) : 32;
  const int gl = (threadIdx.x & 31) % G;
  const int warp = threadIdx.x >> 5;
  const int64_t ncta = a.nchunks / kWarps;
  for (int64_t b = blockIdx.x; b < ncta; b += gridDim.x) {
    const int64_t kb = a.ckb[b];
    const int64_t r0 = kb * kTileRows;
    const int rows = (int)min((int64_t)kTileRows, a.It - r0);
    const double2* src = reinterpret_cast<const double2*>(a.F[NOTHER - 1] + r0 * R);
    __syncthreads();                           // previous block's readers are done
    for (int x = threadIdx.x; x < rows * (R / 2); x += blockDim.x) slab[x] = __ldg(src + x);
    __syncthreads();
    const char* Fb[NOTHER];
#pragma unroll
    for (int q = 0; q < NOTHER - 1; q++) Fb[q] = reinterpret_cast<const char*>(a.F[q]) + gl * 16;
    // slot NOTHER-1 indices are absolute rows: shift the slab base by -r0 rows
    Fb[NOTHER - 1] = reinterpret_cast<const char*>(slab) - r0 * (int64_t)(R * 8) + gl * 16;
    process_chunk<NOTHER, R, RECB>(a, b * kWarps + warp, Fb, srec);
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
    const int64_t p0 = chunk_begin(a, c);
    const int64_t p1 = chunk_end(a, c);
    const int32_t ct = a.cont[c];
    int64_t row = ct >= 0 ? (int64_t)ct : a.lb[c];
    const int64_t row_end = (c == a.nchunks - 1) ? a.I : a.lb[c + 1];
    int64_t seg0 = max(a.rowptr[row < row_end ? row : 0], p0);
    for (; row < row_end; row++) {
      const int64_t seg1 = min(a.rowptr[row + 1], p1);
      const unsigned kbrow = a.pk_rel >= 0 ? (unsigned)(row / a.Iout) * a.pk_blk : 0u;   // block-relative slot
      double acc[CPL];
#pragma unroll
      for (int s = 0; s < CPL; s++) acc[s] = 0.0;
      for (int64_t p = seg0; p < seg1; p++) {
        const char* r = a.rec + p * a.recb;
        const double v = *reinterpret_cast<const double*>(r + a.recb - 8);
        double w[CPL];
        for (int q = 0; q < a.nother; q++) {
          unsigned j = reinterpret_cast<const unsigned*>(r)[q];
          const double* fq = a.F[q];
          if (a.pk) {
            const unsigned f = pk_field(a, q, reinterpret_cast<const unsigned*>(r)[0], reinterpret_cast<const unsigned*>(r)[1]);
            j = f & ~a.pk_hot[q];
            if (f & a.pk_hot[q]) fq = a.HF[q];
            else if (q == a.pk_rel) j += kbrow;
          } else if ((int)j < 0) {
            fq = a.HF[q];                   // hot row (hot-row table)
            j &= 0x7fffffffu;
          }
          const double* src = fq + (size_t)j * (unsigned)R;
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
      double* dst = (ct >= 0 && row == (int64_t)ct) ? a.carry + c * (int64_t)R : a.M + (row - a.rbase) * (int64_t)R;
#pragma unroll
      for (int s = 0; s < CPL; s++)
        if (lane + 32 * s < R) dst[lane + 32 * s] = acc[s];
      seg0 = seg1;
    }
  }
}

// Carry fix-up.  The run of carry chunks of row h is [c0, cend]: c0 = the chunk
// after h's owner, cend = the chunk holding h's last nonzero.  Two levels in a
// fixed order (deterministic): groups of kFixGroup consecutive carries aligned
// at c0 are summed by one warp each, then the group sums of a run are added in
// order to M[h].  Heavy power-law rows (hundreds of carries) are thus spread
// over many warps instead of one.
constexpr int kFixGroup = 16;

__device__ __forceinline__ int64_t chunk_of(int64_t p, int64_t chunk, const int64_t* wstart, int64_t nchunks) {
  if (!wstart) return p / chunk;     // absolute chunk index (subtract the launch's cbase)
  int64_t lo = 0, hi = nchunks - 1;            // last chunk with wstart <= p
  while (lo < hi) {
    const int64_t mid = (lo + hi + 1) >> 1;
    if (wstart[mid] <= p) lo = mid; else hi = mid - 1;
  }
  return lo;
}

__global__ void k_carry_groups(const int32_t* __restrict__ cont, int64_t nchunks, const int64_t* __restrict__ rowptr,
                               int64_t chunk, const int64_t* __restrict__ wstart, int64_t cbase,
                               const double* __restrict__ carry, int R, double* __restrict__ gsum) {
  const int lane = threadIdx.x & 31;
  const int64_t warp0 = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t c = warp0; c < nchunks; c += nwarps) {
    const int32_t h = cont[c];
    if (h < 0) continue;
    const int64_t c0 = chunk_of(rowptr[h], chunk, wstart, nchunks) - cbase + 1;
    if ((c - c0) % kFixGroup != 0) continue;                // not a group leader
    const int64_t cend = min(chunk_of(rowptr[h + 1] - 1, chunk, wstart, nchunks) - cbase, c + kFixGroup - 1);
    for (int col = lane; col < R; col += 32) {
      double s0 = 0.0, s1 = 0.0, s2 = 0.0, s3 = 0.0;
      int64_t cc = c;
      for (; cc + 3 <= cend; cc += 4) {
        s0 += carry[cc * R + col];
        s1 += carry[(cc + 1) * R + col];
        s2 += carry[(cc + 2) * R + col];
        s3 += carry[(cc + 3) * R + col];
      }
      for (; cc <= cend; cc++) s0 += carry[cc * R + col];
      gsum[c * R + col] = (s0 + s1) + (s2 + s3);
    }
  }
}

__global__ void k_carry_fixup(const int32_t* __restrict__ cont, int64_t nchunks, const int64_t* __restrict__ rowptr,
                              int64_t chunk, const int64_t* __restrict__ wstart, int64_t cbase, int64_t rbase,
                              const double* __restrict__ gsum, int R, double* __restrict__ M) {
  const int lane = threadIdx.x & 31;
  const int64_t warp0 = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t c = warp0; c < nchunks; c += nwarps) {
    const int32_t h = cont[c];
    if (h < 0 || (c > 0 && cont[c - 1] == h)) continue;     // run starts only
    const int64_t cend = chunk_of(rowptr[h + 1] - 1, chunk, wstart, nchunks) - cbase;
    for (int col = lane; col < R; col += 32) {
      double s = 0.0;
      for (int64_t cc = c; cc <= cend; cc += kFixGroup) s += gsum[cc * R + col];
      M[((int64_t)h - rbase) * R + col] += s;
    }
  }
}

// M[i, :] = sum over blocks kb (in order) of the partial rows P[kb * I + i, :]; with
// acc, M is the running sum of earlier blocks (a batch of blocks continues it:
// the same summation order as one pass over all blocks)
__global__ void k_reduce_blocks(const double* __restrict__ Pv, int64_t I, int64_t nblk, int R,
                                double* __restrict__ M, int acc) {
  const int64_t n = I * R;
  for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < n;
       x += (int64_t)gridDim.x * blockDim.x) {
    double s = acc ? M[x] : 0.0;
    for (int64_t kb = 0; kb < nblk; kb++) s += Pv[kb * n + x];
    M[x] = s;
  }
}

template <int NOTHER, int RECB, int RR>
bool launch_tiled_r(const MArgs& a, int grid, cudaStream_t st) {
  const size_t smem = (size_t)kTileRows * RR * 8;
  static bool attr = false;
  if (!attr) {
    if (cudaFuncSetAttribute(k_mttkrp_tiled<NOTHER, RR, RECB>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)smem) != cudaSuccess) return false;
    attr = true;
  }
  k_mttkrp_tiled<NOTHER, RR, RECB><<<grid, kWarps * 32, smem, st>>>(a);
  return true;
}

template <int NOTHER, int RECB>
bool launch_fast(const MArgs& a, int grid, cudaStream_t st, bool tiled, int gl, bool hot) {
  // CTAs per SM by nonzeros per row (mttkrp_minb): short rows -- row flushes dominate,
  // latency hiding needs warps -- 4 (64 registers); medium rows (R = 32 / 64) 3 (80);
  // long rows 2 (128)
  const int minb = mttkrp_minb(a.nnz, a.I - a.rbase, a.R, a.l2blocked != 0, hot, NOTHER);
  const bool short_rows = minb == 4;
  const bool mid_rows = minb == 3;
  if constexpr (RECB == 16 && NOTHER == 3) {
    if (a.pk_rel >= 0) {   // packed L2-blocked copy (block-relative slot): R = 32 / 64 kernels, else generic
#define RCASE(RR, GG, HH)                                                                                    \
  if (a.R == RR && gl == GG && hot == HH) {                                                                \
    if (short_rows) k_mttkrp_fast<NOTHER, RR, RECB, 4, GG, HH, 1, true><<<grid, kWarps * 32, 0, st>>>(a);     \
    else k_mttkrp_fast<NOTHER, RR, RECB, 2, GG, HH, 1, true><<<grid, kWarps * 32, 0, st>>>(a);                \
    return true;                                                                                           \
  }
      RCASE(32, 0, false) RCASE(32, 0, true) RCASE(32, 8, false) RCASE(64, 0, false) RCASE(64, 0, true)
#undef RCASE
      return false;
    }
  }
  if (tiled) {
    switch (a.R) {     // slab = 256 rows x R doubles: 2 KB .. 128 KB
      case 8: return launch_tiled_r<NOTHER, RECB, 8>(a, grid, st);
      case 16: return launch_tiled_r<NOTHER, RECB, 16>(a, grid, st);
      case 32: return launch_tiled_r<NOTHER, RECB, 32>(a, grid, st);
      case 64: return launch_tiled_r<NOTHER, RECB, 64>(a, grid, st);
      default: break;  // other ranks: the flat kernel on the k-blocked copy
    }
  }
#define GCASE(RR, GG)                                                                   \
  if (a.R == RR && gl == GG) {                                                      \
    if (short_rows) k_mttkrp_fast<NOTHER, RR, RECB, 4, GG><<<grid, kWarps * 32, 0, st>>>(a); \
    else if (mid_rows) k_mttkrp_fast<NOTHER, RR, RECB, 3, GG><<<grid, kWarps * 32, 0, st>>>(a); \
    else k_mttkrp_fast<NOTHER, RR, RECB, 2, GG><<<grid, kWarps * 32, 0, st>>>(a);          \
    return true;                                                                        \
  }
  GCASE(32, 8) GCASE(64, 16)
#undef GCASE
  // hot-row copies at R = 32: unrolled gathers (mttkrp_unr; 5+ other modes would spill)
  if constexpr (NOTHER <= 4) {
    const int unr = (hot && a.R == 32) ? mttkrp_unr(a.nnz, a.I - a.rbase, a.R, a.l2blocked != 0, hot, NOTHER) : 1;
#define UCASE(UU)                                                                                      \
  if (unr == UU) {                                                                                     \
    if (short_rows) k_mttkrp_fast<NOTHER, 32, RECB, 4, 0, true, UU><<<grid, kWarps * 32, 0, st>>>(a);   \
    else if (mid_rows) k_mttkrp_fast<NOTHER, 32, RECB, 3, 0, true, UU><<<grid, kWarps * 32, 0, st>>>(a); \
    else k_mttkrp_fast<NOTHER, 32, RECB, 2, 0, true, UU><<<grid, kWarps * 32, 0, st>>>(a);              \
    return true;                                                                                       \
  }
    // medium and long rows of hot-row copies (4-mode, R = 32, >= 16 nonzeros per row): 8-lane
    // groups, 4 nonzeros per warp step (mttkrp_hot_g8)
    if constexpr (NOTHER == 3) {
      if (mttkrp_hot_g8(a.nnz, a.I - a.rbase, a.R, a.l2blocked != 0, hot, NOTHER)) {
#define G8CASE(UU)                                                                                        \
  if (unr == UU) {                                                                                        \
    k_mttkrp_fast<NOTHER, 32, RECB, 2, 8, true, UU><<<grid, kWarps * 32, 0, st>>>(a);                       \
    return true;                                                                                          \
  }
        G8CASE(1) G8CASE(2) G8CASE(3) G8CASE(4)
#undef G8CASE
      }
    }
    UCASE(2) UCASE(3) UCASE(4)
#undef UCASE
  }
  if (hot) {           // copies with hot-row slots (large factors): R = 16 / 32 / 64, else generic
    switch (a.R) {
#define HCASE(RR)                                                                              \
  case RR:                                                                                     \
    if (short_rows) k_mttkrp_fast<NOTHER, RR, RECB, 4, 0, true><<<grid, kWarps * 32, 0, st>>>(a); \
    else if (mid_rows) k_mttkrp_fast<NOTHER, RR, RECB, 3, 0, true><<<grid, kWarps * 32, 0, st>>>(a); \
    else k_mttkrp_fast<NOTHER, RR, RECB, 2, 0, true><<<grid, kWarps * 32, 0, st>>>(a);           \
    return true;
      HCASE(16) HCASE(32) HCASE(64)
#undef HCASE
      default: return false;
    }
  }
  switch (a.R) {
#define CASE(RR)                                                                     \
  case RR:                                                                           \
    if (short_rows) k_mttkrp_fast<NOTHER, RR, RECB, 4><<<grid, kWarps * 32, 0, st>>>(a); \
    else k_mttkrp_fast<NOTHER, RR, RECB, 2><<<grid, kWarps * 32, 0, st>>>(a);           \
    return true;
#define CASE3(RR)                                                                    \
  case RR:                                                                           \
    if (short_rows) k_mttkrp_fast<NOTHER, RR, RECB, 4><<<grid, kWarps * 32, 0, st>>>(a); \
    else if (mid_rows) k_mttkrp_fast<NOTHER, RR, RECB, 3><<<grid, kWarps * 32, 0, st>>>(a); \
    else k_mttkrp_fast<NOTHER, RR, RECB, 2><<<grid, kWarps * 32, 0, st>>>(a);           \
    return true;
    CASE(2) CASE(4) CASE(8) CASE(16) CASE3(32) CASE3(64) CASE(128)
#undef CASE
#undef CASE3
    default: return false;
  }
}

cstf_status launch_main(const MArgs& a, int grid, int tgrid, cudaStream_t st, int gl, bool hot = false) {
  bool done = false;
  const bool tl = a.ckb != nullptr;
  const int g = tl ? tgrid : grid;
  if (hot) gl = 0;                 // hot-row copies: the default group width (factors stream from HBM)
  switch (a.nother) {
    case 1: done = launch_fast<1, 16>(a, grid, st, false, gl, hot); break;
    case 2: done = launch_fast<2, 16>(a, g, st, tl, gl, hot); break;
    case 3: done = a.pk ? launch_fast<3, 16>(a, g, st, tl, gl, hot) : launch_fast<3, 32>(a, g, st, tl, gl, hot); break;
    case 4: done = launch_fast<4, 32>(a, g, st, tl, gl, hot); break;
    case 5: done = launch_fast<5, 32>(a, g, st, tl, gl, hot); break;
    case 6: done = launch_fast<6, 32>(a, g, st, tl, gl, hot); break;
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
  DevBuf lb, cont, carry, gsum, partial, kbptr, queue;
  std::vector<int64_t> hk;
};

__global__ void k_kb_offsets(const int64_t* __restrict__ rowptr, int64_t I, int64_t nblk,
                             int64_t* __restrict__ out) {
  for (int64_t b = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; b <= nblk; b += (int64_t)gridDim.x * blockDim.x)
    out[b] = rowptr[b * I];
}
Workspace& ws() {
  static thread_local Workspace w[64];
  int dev = 0;
  cudaGetDevice(&dev);
  return w[dev & 63];
}

// Work split of a k-blocked copy (host logic, cached on the mode store): every
// block's nonzero range is cut into CTA chunks of <= kCtaChunk nonzeros, each
// split into kWarps warp chunks; every block gets at least one CTA chunk so its
// (possibly empty) partial rows are written.
constexpr int64_t kCtaChunk = 16384;

cstf_status tiled_split(const ModeStore& ms, cudaStream_t st) {
  if (ms.nctachunks > 0) return CSTF_OK;
  Workspace& w = ws();
  CSTF_TRY(w.kbptr.ensure((size_t)(ms.nblk + 1) * 8));
  k_kb_offsets<<<(int)((ms.nblk + 256) / 256), 256, 0, st>>>(ms.rowptr.as<int64_t>(), ms.I, ms.nblk,
                                                             w.kbptr.as<int64_t>());
  CSTF_LAUNCHED();
  std::vector<int64_t> kp((size_t)ms.nblk + 1);
  CSTF_CUDA(cudaMemcpyAsync(kp.data(), w.kbptr.p, kp.size() * 8, cudaMemcpyDeviceToHost, st));
  CSTF_CUDA(cudaStreamSynchronize(st));
  std::vector<int64_t> starts;
  std::vector<int32_t> kbs;
  for (int64_t b = 0; b < ms.nblk; b++) {
    const int64_t lo = kp[(size_t)b], hi = kp[(size_t)b + 1];
    const int64_t nc = std::max<int64_t>(1, (hi - lo + kCtaChunk - 1) / kCtaChunk);
    for (int64_t k = 0; k < nc; k++) {
      const int64_t c0 = lo + (hi - lo) * k / nc, c1 = lo + (hi - lo) * (k + 1) / nc;
      kbs.push_back((int32_t)b);
      for (int wv = 0; wv < kWarps; wv++) starts.push_back(c0 + (c1 - c0) * wv / kWarps);
    }
  }
  starts.push_back(ms.nnz);
  CSTF_TRY(ms.wstart.alloc(starts.size() * 8));
  CSTF_TRY(ms.ckb.alloc(kbs.size() * 4));
  CSTF_CUDA(cudaMemcpyAsync(ms.wstart.p, starts.data(), starts.size() * 8, cudaMemcpyHostToDevice, st));
  CSTF_CUDA(cudaMemcpyAsync(ms.ckb.p, kbs.data(), kbs.size() * 4, cudaMemcpyHostToDevice, st));
  CSTF_CUDA(cudaStreamSynchronize(st));
  ms.nctachunks = (int64_t)kbs.size();
  ms.nwchunks = ms.nctachunks * kWarps;
  return CSTF_OK;
}

// L2-blocked copy: nonzeros ordered by (block of the
// blocked factor's row, output row, ...).  Blocks are processed in batches whose
// partial rows fit a workspace budget -- a quarter of the device memory, a
// function of the device and the problem only, so results are deterministic
// (CSTF_L2_BATCH_BYTES overrides; halved only if the allocation fails).  Every
// batch is one launch over its own nonzero range with chunks taken from a global
// counter in copy order, so the nonzeros in flight touch a narrow slice of the
// blocked factor (its L2-resident slab); its partials continue the running sum of
// M in block order.
cstf_status mttkrp_l2_blocked(const ModeStore& ms, MArgs& a, int R, int gl, double* d_M, cudaStream_t st,
                              int64_t* nl, bool hot) {
  const DeviceInfo& di = device_info();
  Workspace& w = ws();
  const int64_t I = ms.I, nblk = ms.nblk, nnz = ms.nnz;
  if ((int64_t)ms.kp.size() != nblk + 1) {           // block boundaries (host copy, cached)
    CSTF_TRY(w.kbptr.ensure((size_t)(nblk + 1) * 8));
    k_kb_offsets<<<(int)((nblk + 256) / 256), 256, 0, st>>>(ms.rowptr.as<int64_t>(), I, nblk, w.kbptr.as<int64_t>());
    CSTF_LAUNCHED();
    (*nl)++;
    ms.kp.resize((size_t)nblk + 1);
    CSTF_CUDA(cudaMemcpyAsync(ms.kp.data(), w.kbptr.p, ms.kp.size() * 8, cudaMemcpyDeviceToHost, st));
    CSTF_CUDA(cudaStreamSynchronize(st));
  }
  const size_t per_block = (size_t)I * R * 8;
  size_t budget = 0;
  if (const char* be = getenv("CSTF_L2_BATCH_BYTES")) {
    budget = (size_t)atoll(be);
  } else {
    // at most a quarter of the device and half of what is free (counting the buffer
    // already cached); the summation order does not depend on the batch size (each
    // batch continues M's running sum in block order), so neither do the results
    size_t fr = 0, tot = 0;
    CSTF_CUDA(cudaMemGetInfo(&fr, &tot));
    budget = std::min(tot / 4, (fr + w.partial.bytes) / 2);
  }
  int64_t B = std::max<int64_t>(1, std::min<int64_t>(nblk, (int64_t)(budget / std::max<size_t>(per_block, 1))));
  while (w.partial.ensure((size_t)B * per_block) != CSTF_OK) {
    if (B == 1) return fail(CSTF_ERR_OUT_OF_MEMORY, "MTTKRP partial rows of one L2 block (set CSTF_L2_BLOCK=0)");
    B = (B + 1) / 2;
  }
  const int ctas = di.sms * mttkrp_minb(nnz, ms.Ivirt, R, true, hot, a.nother);   // resident CTAs only (= launch_fast's budget)
  a.l2blocked = 1;
  // chunk: the window in flight (resident warps x chunk) about half a block
  int64_t chunk = (nnz / std::max<int64_t>(nblk, 1)) / (2 * (int64_t)ctas * kWarps);
  chunk = std::min<int64_t>(1024, std::max<int64_t>(256, (chunk + 31) / 32 * 32));
  if (const char* ce = getenv("CSTF_L2_CHUNK"))
    if (atoll(ce) >= 32) chunk = (atoll(ce) + 31) / 32 * 32;
  CSTF_TRY(w.queue.ensure(8));
  double* part = w.partial.as<double>();
  // Large blocks (>= 16M nonzeros, Amazon): one launch per block with the block's
  // slab as a persisting L2 access window (64 MB set-aside, capped by the device),
  // so the other factor's random rows do not evict it (Amazon 184/189/200 ->
  // 175/175/183 ms per mode).  (Deterministic: the launches follow the blocks.)
  // The set-aside is reserved once per device; L2
  // lines not claimed by persisting accesses stay usable by all other traffic.
  // CSTF_L2_PERSIST=<bytes> overrides (0 disables).
  size_t persist = (nnz / std::max<int64_t>(nblk, 1) >= ((int64_t)16 << 20)) ? ((size_t)64 << 20) : 0;
  if (const char* pe = getenv("CSTF_L2_PERSIST")) persist = (size_t)atoll(pe);
  // The caller's persisting-L2 limit and the stream's access-policy window are saved
  // here and restored after the blocked launches (no process-wide state
  // left changed by a stream-ordered library call).
  size_t saved_limit = 0;
  cudaStreamAttrValue saved_win = {};
  bool restore_limit = false, restore_win = false;
  if (persist) {
    int maxp = 0;
    cudaDeviceGetAttribute(&maxp, cudaDevAttrMaxPersistingL2CacheSize, di.device);
    persist = std::min<size_t>(persist, (size_t)std::max(maxp, 0));
    if (persist && cudaDeviceGetLimit(&saved_limit, cudaLimitPersistingL2CacheSize) != cudaSuccess) {
      cudaGetLastError();
      persist = 0;
    }
    if (persist && saved_limit != persist) {
      if (cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, persist) == cudaSuccess) {
        restore_limit = true;
      } else {                    // not available (e.g. MIG): plain launches, no error
        cudaGetLastError();
        persist = 0;
      }
    }
    if (persist) {
      if (cudaStreamGetAttribute(st, cudaStreamAttributeAccessPolicyWindow, &saved_win) == cudaSuccess)
        restore_win = true;
      else
        cudaGetLastError();
    }
  }
  for (int64_t b0 = 0; b0 < nblk; b0 += B) {
    const int64_t b1 = std::min(nblk, b0 + B);
    const int64_t ustep = persist ? 1 : b1 - b0;
    for (int64_t u0 = b0; u0 < b1; u0 += ustep) {
      const int64_t u1 = std::min(b1, u0 + ustep);
      const int64_t pbase = ms.kp[(size_t)u0], pend = ms.kp[(size_t)u1];
      const int64_t rbase = u0 * I, rend = u1 * I;
      const int64_t n = pend - pbase;
      const int64_t cbase = pbase / chunk;
      const int64_t nchunks = n > 0 ? (pend + chunk - 1) / chunk - cbase : 1;
      CSTF_TRY(w.carry.ensure((size_t)nchunks * R * 8));
      CSTF_TRY(w.gsum.ensure((size_t)nchunks * R * 8));
      CSTF_TRY(w.lb.ensure((size_t)(nchunks + 1) * 8));
      CSTF_TRY(w.cont.ensure((size_t)nchunks * 4));
      const int gb = (int)std::min<int64_t>((nchunks + 1 + 255) / 256, (int64_t)di.sms * 8);
      k_chunk_bounds<<<gb, 256, 0, st>>>(a.rowptr, rbase, rend, pbase, pend, chunk, cbase, nchunks, nullptr,
                                          w.lb.as<int64_t>(), w.cont.as<int32_t>());
      CSTF_LAUNCHED();
      double* upart = part + (size_t)(u0 - b0) * I * R;
      a.pbase = pbase;
      a.cbase = cbase;
      a.rbase = rbase;
      a.I = rend;
      a.nnz = n;
      a.chunk = chunk;
      a.nchunks = nchunks;
      a.lb = w.lb.as<int64_t>();
      a.cont = w.cont.as<int32_t>();
      a.M = upart;
      a.carry = w.carry.as<double>();
      a.queue = nullptr;
      if (nchunks > 1) {
        CSTF_CUDA(cudaMemsetAsync(w.queue.p, 0, 8, st));
        a.queue = w.queue.as<unsigned long long>();
      }
      if (persist) {
        const int64_t r0 = u0 * ms.blk_rows;
        const int64_t nr = std::min<int64_t>(ms.blk_rows * (u1 - u0), a.It_blk - r0);
        cudaStreamAttrValue v = {};
        v.accessPolicyWindow.base_ptr = const_cast<double*>(a.F[ms.tslot] + r0 * R);
        v.accessPolicyWindow.num_bytes = (size_t)std::max<int64_t>(nr, 0) * R * 8;
        v.accessPolicyWindow.hitRatio = std::min(1.0f, (float)persist / (float)std::max<size_t>(v.accessPolicyWindow.num_bytes, 1));
        v.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
        v.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
        if (cudaStreamSetAttribute(st, cudaStreamAttributeAccessPolicyWindow, &v) != cudaSuccess) cudaGetLastError();
      }
      const int grid = (int)std::min<int64_t>((nchunks + kWarps - 1) / kWarps, (int64_t)ctas);
      CSTF_TRY(launch_main(a, grid, grid, st, gl, hot));
      *nl += 2;
      if (nchunks > 1) {
        const int g = (int)std::min<int64_t>((nchunks * 32 + 255) / 256, (int64_t)di.sms * 8);
        k_carry_groups<<<g, 256, 0, st>>>(a.cont, nchunks, a.rowptr, chunk, nullptr, cbase, a.carry, R,
                                          w.gsum.as<double>());
        CSTF_LAUNCHED();
        k_carry_fixup<<<g, 256, 0, st>>>(a.cont, nchunks, a.rowptr, chunk, nullptr, cbase, rbase,
                                         w.gsum.as<double>(), R, upart);
        CSTF_LAUNCHED();
        *nl += 2;
      }
    }
    const int64_t nm = I * R;
    const int g = (int)std::min<int64_t>((nm + 255) / 256, (int64_t)di.sms * 16);
    k_reduce_blocks<<<g, 256, 0, st>>>(part, I, b1 - b0, R, d_M, b0 > 0 ? 1 : 0);
    CSTF_LAUNCHED();
    (*nl)++;
  }
  if (persist) {
    // restore the caller's window; once the launches have run, release the persisting
    // lines (cudaCtxResetPersistingL2Cache is not stream-ordered, hence the one host
    // synchronisation of this path) and restore the caller's set-aside
    cudaStreamAttrValue v = {};
    if (restore_win) v = saved_win;
    else v.accessPolicyWindow.num_bytes = 0;
    if (cudaStreamSetAttribute(st, cudaStreamAttributeAccessPolicyWindow, &v) != cudaSuccess) cudaGetLastError();
    CSTF_CUDA(cudaStreamSynchronize(st));
    if (cudaCtxResetPersistingL2Cache() != cudaSuccess) cudaGetLastError();
    if (restore_limit && cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, saved_limit) != cudaSuccess)
      cudaGetLastError();
  }
  return CSTF_OK;
}

}  // namespace

// tab[s, :] = F[rows[s], :] for the hot slots of one factor
__global__ void k_hot_refresh(const double* __restrict__ F, const int32_t* __restrict__ rows, int64_t H, int R,
                              double* __restrict__ tab) {
  const int64_t n = H * R;
  for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < n; x += (int64_t)gridDim.x * blockDim.x) {
    const int64_t s = x / R, c = x % R;
    tab[x] = F[(int64_t)rows[s] * R + c];
  }
}

cstf_status hot_refresh(const cstf_tensor* X, int k, const double* d_F, int R, cudaStream_t st) {
  if (X->hot_cnt[k] == 0) return CSTF_OK;
  if (X->hot_R != R || !X->hot_tab.p) {
    CSTF_TRY(X->hot_tab.alloc((size_t)X->hot_total * R * 8));
    X->hot_R = R;
  }
  const int64_t n = X->hot_cnt[k] * R;
  const int g = (int)std::min<int64_t>((n + 255) / 256, (int64_t)device_info().sms * 16);
  k_hot_refresh<<<g, 256, 0, st>>>(d_F, X->hot_rows.as<int32_t>() + X->hot_off[k], X->hot_cnt[k], R,
                                   X->hot_tab.as<double>() + X->hot_off[k] * R);
  CSTF_LAUNCHED();
  return CSTF_OK;
}

// The persisting-L2 set-aside the hot-row window needs: the device maximum (the
// caller's limit is saved and restored by hot_persist_end, which also releases the
// persisting lines; call it after a stream synchronisation).
cstf_status hot_persist_begin(const cstf_tensor* X, L2Persist& p) {
  p.active = false;
  if (X->hot_total == 0 || (getenv("CSTF_HOT_WINDOW") && atoi(getenv("CSTF_HOT_WINDOW")) == 0)) return CSTF_OK;
  int maxp = 0;
  cudaDeviceGetAttribute(&maxp, cudaDevAttrMaxPersistingL2CacheSize, device_info().device);
  if (maxp <= 0 || cudaDeviceGetLimit(&p.saved, cudaLimitPersistingL2CacheSize) != cudaSuccess) {
    cudaGetLastError();
    return CSTF_OK;
  }
  if (p.saved != (size_t)maxp && cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, (size_t)maxp) != cudaSuccess) {
    cudaGetLastError();               // not available (e.g. MIG): hot tables without persistence
    return CSTF_OK;
  }
  p.active = true;
  return CSTF_OK;
}

void hot_persist_end(L2Persist& p) {
  if (!p.active) return;
  if (cudaCtxResetPersistingL2Cache() != cudaSuccess) cudaGetLastError();
  if (cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, p.saved) != cudaSuccess) cudaGetLastError();
  p.active = false;
}

void release_mttkrp_ws() {
  Workspace& w = ws();
  for (DevBuf* b : {&w.lb, &w.cont, &w.carry, &w.gsum, &w.partial, &w.kbptr, &w.queue}) b->release();
}

cstf_status mttkrp(const cstf_tensor* X, int mode, int R, const double* const* d_factors,
                   double* d_M, cudaStream_t st, int64_t* launches, bool hot_fresh) {
  const ModeStore& ms = X->mode[mode];
  const int N = X->N;
  const DeviceInfo& di = device_info();
  const int64_t nnz = ms.nnz;
  Workspace& w = ws();
  if (ms.I == 0) return CSTF_OK;
  MArgs a;
  a.wstart = nullptr;
  a.ckb = nullptr;
  a.queue = nullptr;
  a.l2blocked = 0;
  a.pbase = 0;
  a.cbase = 0;
  a.rbase = 0;
  a.rowptr = ms.rowptr.as<int64_t>();
  a.rec = ms.rec.as<char>();
  a.recb = ms.recb;
  a.pk = ms.pk ? 1 : 0;
  for (int q = 0; q < 3; q++) { a.pk_sh[q] = ms.pk_sh[q]; a.pk_mask[q] = ms.pk_mask[q]; a.pk_hot[q] = ms.pk_hot[q]; }
  a.pk_rel = ms.pk_rel;
  a.pk_blk = ms.pk_rel >= 0 ? (uint32_t)ms.blk_rows : 1u;
  a.Iout = ms.I > 0 ? ms.I : 1;
  a.nother = N - 1;
  for (int q = 0; q < N - 1; q++) a.F[q] = d_factors[ms.other[q]];
  a.It = X->dims[ms.other[N - 2]];      // slab blocks: rows of the last slot's factor
  a.It_blk = X->partitioned ? (int64_t)X->nranks * X->rows_per_rank[ms.other[ms.tslot]] : X->dims[ms.other[ms.tslot]];
  a.R = R;
  for (int q = 0; q < 7; q++) a.HF[q] = nullptr;
  // Hot-row tables: refresh from the caller's factors unless the caller keeps them
  // current (factorize), then read the hot rows under a persisting access window
  // over the whole table (the caller's window is restored after the launches).
  const bool hot = ms.hotmask != 0 && X->hot_total > 0;
  L2Persist own;
  cudaStreamAttrValue saved_win = {};
  bool win_set = false;
  if (hot) {
    for (int q = 0; q < N - 1; q++)
      if (ms.hotmask & (1 << q)) {
        if (!hot_fresh || X->hot_R != R) CSTF_TRY(hot_refresh(X, ms.other[q], d_factors[ms.other[q]], R, st));
      }
    for (int q = 0; q < N - 1; q++)
      if (ms.hotmask & (1 << q)) a.HF[q] = X->hot_tab.as<double>() + X->hot_off[ms.other[q]] * R;
    if (!hot_fresh) CSTF_TRY(hot_persist_begin(X, own));
    int maxw = 0;
    cudaDeviceGetAttribute(&maxw, cudaDevAttrMaxAccessPolicyWindowSize, di.device);
    const bool persist_on = hot_fresh ? !(getenv("CSTF_HOT_WINDOW") && atoi(getenv("CSTF_HOT_WINDOW")) == 0)
                                      : own.active;
    if (persist_on && maxw > 0 && cudaStreamGetAttribute(st, cudaStreamAttributeAccessPolicyWindow, &saved_win) == cudaSuccess) {
      cudaStreamAttrValue v = {};
      v.accessPolicyWindow.base_ptr = X->hot_tab.p;
      v.accessPolicyWindow.num_bytes = std::min<size_t>((size_t)X->hot_total * R * 8, (size_t)maxw);
      v.accessPolicyWindow.hitRatio = 1.0f;
      v.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
      v.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
      if (cudaStreamSetAttribute(st, cudaStreamAttributeAccessPolicyWindow, &v) == cudaSuccess) win_set = true;
      else cudaGetLastError();
    } else {
      cudaGetLastError();
    }
  }
  // after the launches: the caller's window back; a standalone call also releases the
  // persisting lines and the set-aside (one host synchronisation)
  auto hot_done = [&]() -> cstf_status {
    if (win_set && cudaStreamSetAttribute(st, cudaStreamAttributeAccessPolicyWindow, &saved_win) != cudaSuccess)
      cudaGetLastError();
    if (own.active) {
      CSTF_CUDA(cudaStreamSynchronize(st));
      hot_persist_end(own);
    }
    return CSTF_OK;
  };
  // Lanes per factor row: 8 lanes x 32 B (4 nonzeros per warp step) when the gathered
  // factors are L2-resident -- more nonzeros per load instruction, so adjacent
  // fiber nonzeros share L1 wavefronts (NELL-2 1.80 -> 1.63 ms per mode); the
  // default 16 lanes x 16 B when they stream from HBM (Delicious, Amazon: no gain
  // or a loss).  CSTF_MTTKRP_G forces a value (experiments).
  int gl = 0;
  {
    int64_t gbytes = 0;
    for (int q = 0; q < N - 1; q++) gbytes += X->dims[ms.other[q]] * (int64_t)R * 8;
    if (R == 32 && gbytes <= (int64_t)di.l2) gl = 8;
    const char* ge = getenv("CSTF_MTTKRP_G");        // read per call (tests force both paths)
    if (ge && (atoi(ge) == 0 || atoi(ge) == 8)) gl = atoi(ge);
  }
  int64_t nl = 0;
  if (ms.tiled && !ms.slab) {
    const cstf_status sb = mttkrp_l2_blocked(ms, a, R, gl, d_M, st, &nl, hot);
    CSTF_TRY(hot_done());
    CSTF_TRY(sb);
    if (launches) *launches += nl;
    return CSTF_OK;
  }
  int64_t chunk = 0, nchunks = 0;
  if (ms.tiled && ms.slab) {
    CSTF_TRY(tiled_split(ms, st));
    nchunks = ms.nwchunks;
    a.wstart = ms.wstart.as<int64_t>();
    a.ckb = ms.ckb.as<int32_t>();
  } else {
    // chunk: ~4 chunks per resident warp, multiple of 32, in [256, 8192]
    const int64_t resident = (int64_t)di.sms * 8 * kWarps;
    chunk = (nnz + resident * 4 - 1) / (resident * 4);
    chunk = ((chunk + 31) / 32) * 32;
    if (chunk < 256) chunk = 256;
    if (chunk > 8192) chunk = 8192;
    nchunks = nnz > 0 ? (nnz + chunk - 1) / chunk : 1;
  }
  CSTF_TRY(w.carry.ensure((size_t)nchunks * R * 8));
  CSTF_TRY(w.gsum.ensure((size_t)nchunks * R * 8));
  const bool fresh = ms.cchunk != chunk || ms.cnchunks != nchunks;   // boundaries cached per mode
  if (fresh) {
    CSTF_TRY(ms.clb.alloc((size_t)(nchunks + 1) * 8));
    CSTF_TRY(ms.ccont.alloc((size_t)nchunks * 4));
  }
  double* out = d_M;
  if (ms.tiled) {
    CSTF_TRY(w.partial.ensure((size_t)ms.Ivirt * R * 8));
    out = w.partial.as<double>();
  }
  a.I = ms.Ivirt;
  a.nnz = nnz;
  a.chunk = chunk;
  a.nchunks = nchunks;
  a.lb = ms.clb.as<int64_t>();
  a.cont = ms.ccont.as<int32_t>();
  a.M = out;
  a.carry = w.carry.as<double>();
  if (fresh) {
    const int g = (int)std::min<int64_t>((nchunks + 1 + 255) / 256, (int64_t)di.sms * 8);
    k_chunk_bounds<<<g, 256, 0, st>>>(a.rowptr, 0, ms.Ivirt, 0, nnz, chunk, 0, nchunks, a.wstart,
                                       ms.clb.as<int64_t>(), ms.ccont.as<int32_t>());
    CSTF_LAUNCHED();
    nl++;
    ms.cchunk = chunk;
    ms.cnchunks = nchunks;
  }
  int grid = (int)std::min<int64_t>((nchunks + kWarps - 1) / kWarps, (int64_t)di.sms * 8);
  const int tgrid = (int)std::min<int64_t>(std::max<int64_t>(ms.nctachunks, 1), (int64_t)di.sms * 2);
  // Chunks in copy order from a global counter, one wave of resident CTAs (the fast
  // kernel's register budget: 2 CTAs/SM for long rows, 4 for short ones): the
  // chunks in flight are neighbours in the copy and no wave tail remains
  // (NELL-2 1.62 -> 1.57 ms per mode, Delicious mode 2 13.1 -> 12.3 ms).
  // Which warp runs a chunk does not change its arithmetic.  CSTF_MTTKRP_QUEUE=0:
  // static grid-stride order.
  {
    const char* qe = getenv("CSTF_MTTKRP_QUEUE");
    const bool pow2 = R >= 2 && R <= 128 && (R & (R - 1)) == 0;
    if (!(qe && atoi(qe) == 0) && !ms.tiled && nchunks > 1 && pow2 && N - 1 <= 6) {
      CSTF_TRY(w.queue.ensure(8));
      CSTF_CUDA(cudaMemsetAsync(w.queue.p, 0, 8, st));
      a.queue = w.queue.as<unsigned long long>();
      grid = std::min(grid, di.sms * mttkrp_minb(nnz, ms.Ivirt, R, false, hot, N - 1));
    }
  }
  {
    const cstf_status sl = launch_main(a, grid, tgrid, st, gl, hot);
    CSTF_TRY(hot_done());
    CSTF_TRY(sl);
  }
  nl++;
  if (nchunks > 1) {
    const int g = (int)std::min<int64_t>((nchunks * 32 + 255) / 256, (int64_t)di.sms * 8);
    k_carry_groups<<<g, 256, 0, st>>>(a.cont, nchunks, a.rowptr, chunk, a.wstart, 0, a.carry, R,
                                      w.gsum.as<double>());
    CSTF_LAUNCHED();
    k_carry_fixup<<<g, 256, 0, st>>>(a.cont, nchunks, a.rowptr, chunk, a.wstart, 0, 0, w.gsum.as<double>(), R, out);
    CSTF_LAUNCHED();
    nl += 2;
  }
  if (ms.tiled) {
    const int64_t n = ms.I * R;
    const int g = (int)std::min<int64_t>((n + 255) / 256, (int64_t)di.sms * 16);
    k_reduce_blocks<<<g, 256, 0, st>>>(out, ms.I, ms.nblk, R, d_M, 0);
    CSTF_LAUNCHED();
    nl++;
  }
  if (launches) *launches += nl;
  return CSTF_OK;
}

}  // namespace cstf
