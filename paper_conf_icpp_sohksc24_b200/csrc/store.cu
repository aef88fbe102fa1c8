// Mode-sorted nonzero store (hot-path step a0).
//
// Host COO -> device -> validate -> canonical order (lexicographic by
// (i_1..i_N), LSD radix sort over <=64-bit packed mode groups, stable so
// duplicates keep input order) -> duplicates summed left to right in input
// order (bit-exact with the oracle's O1) -> ||X||^2 and canonical checksum ->
// for every mode n a copy stably sorted by i_n with an int64 row pointer.
// The element-wise MTTKRP definition this store serves is PAPER.md Fig. 2
// (L403-430); the paper's own format (BLCO, L439-442) is replaced.
#include <cub/cub.cuh>

#include <algorithm>
#include <functional>
#include <cstdlib>
#include <cstring>
#include <vector>

#include "internal.h"

namespace cstf {
namespace {

constexpr int kThreads = 256;
constexpr int kFixedBlocks = 1024;  // fixed => deterministic reductions

inline int grid_for(int64_t n, int threads = kThreads) {
  int64_t g = (n + threads - 1) / threads;
  int cap = device_info().sms * 32;
  if (g > cap) g = cap;
  return (int)(g < 1 ? 1 : g);
}

int bits_for(int64_t dim) {
  int b = 0;
  while (b < 63 && ((int64_t)1 << b) < dim) b++;
  return b;  // dim == 1 -> 0 bits
}

__global__ void k_count_invalid(const int32_t* __restrict__ idx, int64_t n, int64_t dim,
                                unsigned long long* bad) {
  unsigned long long c = 0;
  for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < n;
       p += (int64_t)gridDim.x * blockDim.x) {
    int32_t v = idx[p];
    c += (v < 0 || (int64_t)v >= dim) ? 1ull : 0ull;
  }
  if (c) atomicAdd(bad, c);
}

struct PackArgs {
  const int32_t* idx[8];
  int shift[8];
  int count;
};

// key[p] = packed indices of the group's modes for the nonzero perm[p] (or p when perm == null)
__global__ void k_pack_keys(PackArgs a, const uint32_t* __restrict__ perm, int64_t n,
                            uint64_t* __restrict__ key) {
  for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < n;
       p += (int64_t)gridDim.x * blockDim.x) {
    uint64_t src = perm ? perm[p] : (uint64_t)p;
    uint64_t k = 0;
    for (int m = 0; m < a.count; m++) k |= (uint64_t)(uint32_t)a.idx[m][src] << a.shift[m];
    key[p] = k;
  }
}

__global__ void k_iota(uint32_t* __restrict__ out, int64_t n) {
  for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < n;
       p += (int64_t)gridDim.x * blockDim.x)
    out[p] = (uint32_t)p;
}

template <class T>
__global__ void k_gather(const T* __restrict__ in, const uint32_t* __restrict__ perm, int64_t n,
                         T* __restrict__ out) {
  for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < n;
       p += (int64_t)gridDim.x * blockDim.x)
    out[p] = in[perm[p]];
}

struct IdxArgs {
  const int32_t* idx[8];
  int N;
};

__global__ void k_heads(IdxArgs a, int64_t n, uint32_t* __restrict__ head) {
  for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < n;
       p += (int64_t)gridDim.x * blockDim.x) {
    uint32_t h = (p == 0);
    if (!h)
      for (int m = 0; m < a.N; m++) h |= (a.idx[m][p] != a.idx[m][p - 1]);
    head[p] = h;
  }
}

// segid = inclusive scan of heads (1-based); start[segid-1] = p at heads
__global__ void k_seg_starts(const uint32_t* __restrict__ head, const uint32_t* __restrict__ segid,
                             int64_t n, uint32_t* __restrict__ start) {
  for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < n;
       p += (int64_t)gridDim.x * blockDim.x)
    if (head[p]) start[segid[p] - 1] = (uint32_t)p;
}

struct OutArgs {
  int32_t* idx[8];
  int N;
};

// one thread per coalesced entry: left-to-right sum of the duplicates (input order)
__global__ void k_coalesce(IdxArgs in, const double* __restrict__ vals,
                           const uint32_t* __restrict__ start, int64_t nseg, int64_t n,
                           OutArgs out, double* __restrict__ out_vals) {
  for (int64_t s = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; s < nseg;
       s += (int64_t)gridDim.x * blockDim.x) {
    int64_t p0 = start[s];
    int64_t p1 = (s + 1 < nseg) ? (int64_t)start[s + 1] : n;
    double v = vals[p0];
    for (int64_t p = p0 + 1; p < p1; p++) v = __dadd_rn(v, vals[p]);
    out_vals[s] = v;
    for (int m = 0; m < in.N; m++) out.idx[m][s] = in.idx[m][p0];
  }
}

__device__ __forceinline__ uint64_t mix64(uint64_t z) {
  z ^= z >> 30; z *= 0xBF58476D1CE4E5B9ULL;
  z ^= z >> 27; z *= 0x94D049BB133111EBULL;
  z ^= z >> 31; return z;
}

// Per fixed block: partial sum of v^2 (tree order) and of the entry checksums (mod 2^64).
__global__ void __launch_bounds__(kThreads) k_norm_hash(IdxArgs a, const double* __restrict__ vals,
                                                        int64_t n, double* __restrict__ part_norm,
                                                        unsigned long long* __restrict__ part_hash) {
  __shared__ double sn[kThreads];
  __shared__ unsigned long long sh[kThreads];
  double acc = 0.0;
  unsigned long long h = 0;
  for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < n;
       p += (int64_t)gridDim.x * blockDim.x) {
    double v = vals[p];
    acc = fma(v, v, acc);
    uint64_t z = (uint64_t)p + 1;
    for (int m = 0; m < a.N; m++)
      z = mix64(z ^ ((uint64_t)(uint32_t)a.idx[m][p] + (uint64_t)(m + 1) * 0x9E3779B97F4A7C15ULL));
    z = mix64(z ^ (uint64_t)__double_as_longlong(v));
    h += z;
  }
  sn[threadIdx.x] = acc;
  sh[threadIdx.x] = h;
  __syncthreads();
  for (int s = kThreads / 2; s > 0; s >>= 1) {
    if (threadIdx.x < s) {
      sn[threadIdx.x] += sn[threadIdx.x + s];
      sh[threadIdx.x] += sh[threadIdx.x + s];
    }
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    part_norm[blockIdx.x] = sn[0];
    part_hash[blockIdx.x] = sh[0];
  }
}

__global__ void k_norm_hash_final(const double* __restrict__ part_norm,
                                  const unsigned long long* __restrict__ part_hash, int nb,
                                  double* out_norm, unsigned long long* out_hash) {
  if (threadIdx.x == 0 && blockIdx.x == 0) {
    double s = 0.0;
    unsigned long long h = 0;
    for (int b = 0; b < nb; b++) { s += part_norm[b]; h += part_hash[b]; }
    *out_norm = s;
    *out_hash = h;
  }
}

__global__ void k_histogram(const int32_t* __restrict__ key, int64_t n,
                            unsigned long long* __restrict__ cnt) {
  for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < n;
       p += (int64_t)gridDim.x * blockDim.x)
    atomicAdd(&cnt[key[p]], 1ull);
}

// out[p] = row of p (virtual row v -> v mod I)
__global__ void k_expand_rows(const int64_t* __restrict__ rowptr, int64_t Iv, int64_t I,
                              int32_t* __restrict__ out, int32_t* __restrict__ kbout) {
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < Iv;
       v += (int64_t)gridDim.x * blockDim.x)
    for (int64_t p = rowptr[v]; p < rowptr[v + 1]; p++) {
      out[p] = (int32_t)(v % I);
      if (kbout) kbout[p] = (int32_t)(v / I);      // block of the virtual row
    }
}

// Stable LSD radix sort of positions 0..n-1 by the key tuple keys[0..nk-1]
// (keys[0] most significant).  Keys are packed into <= 64-bit groups from the
// least significant end; every pass is a stable CUB radix sort, so equal
// tuples keep their input order.  Result in `perm` (uint32[n]).
cstf_status lsd_sort(const int32_t* const* keys, const int64_t* dims, int nk, int64_t n, DevBuf& perm,
                     DevBuf& tmp, cudaStream_t st) {
  CSTF_TRY(perm.alloc((size_t)n * 4));
  if (n == 0) return CSTF_OK;
  DevBuf perm_b, key_a, key_b;
  CSTF_TRY(perm_b.alloc((size_t)n * 4));
  CSTF_TRY(key_a.alloc((size_t)n * 8));
  CSTF_TRY(key_b.alloc((size_t)n * 8));
  k_iota<<<grid_for(n), kThreads, 0, st>>>(perm.as<uint32_t>(), n);
  CSTF_LAUNCHED();
  int hi = nk - 1;
  while (hi >= 0) {
    int lo = hi, tot = bits_for(dims[hi]);
    while (lo - 1 >= 0 && tot + bits_for(dims[lo - 1]) <= 64) { lo--; tot += bits_for(dims[lo]); }
    PackArgs pa;
    pa.count = hi - lo + 1;
    int sh = 0;
    for (int m = hi; m >= lo; m--) {
      pa.idx[m - lo] = keys[m];
      pa.shift[m - lo] = sh;
      sh += bits_for(dims[m]);
    }
    if (tot > 0) {
      k_pack_keys<<<grid_for(n), kThreads, 0, st>>>(pa, perm.as<uint32_t>(), n, key_a.as<uint64_t>());
      CSTF_LAUNCHED();
      size_t tb = 0;
      CSTF_CUDA(cub::DeviceRadixSort::SortPairs(nullptr, tb, key_a.as<uint64_t>(), key_b.as<uint64_t>(),
                                                perm.as<uint32_t>(), perm_b.as<uint32_t>(), n, 0, tot, st));
      CSTF_TRY(tmp.ensure(tb));
      CSTF_CUDA(cub::DeviceRadixSort::SortPairs(tmp.p, tb, key_a.as<uint64_t>(), key_b.as<uint64_t>(),
                                                perm.as<uint32_t>(), perm_b.as<uint32_t>(), n, 0, tot, st));
      count_launch();
      std::swap(perm, perm_b);
    }
    hi = lo - 1;
  }
  CSTF_CUDA(cudaStreamSynchronize(st));
  return CSTF_OK;
}

__global__ void k_block_keys(const int32_t* __restrict__ idx_t, const int32_t* __restrict__ idx_n, int64_t n,
                             int64_t I, int64_t blk, int32_t* __restrict__ kb, int32_t* __restrict__ vrow) {
  for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < n;
       p += (int64_t)gridDim.x * blockDim.x) {
    const int32_t b = (int32_t)(idx_t[p] / blk);
    kb[p] = b;
    vrow[p] = (int32_t)((int64_t)b * I + idx_n[p]);
  }
}

// out[p] = lab[in[p]]
__global__ void k_map(const int32_t* __restrict__ in, const int32_t* __restrict__ lab, int64_t n,
                      int32_t* __restrict__ out) {
  for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < n;
       p += (int64_t)gridDim.x * blockDim.x)
    out[p] = lab[in[p]];
}

// positions p whose internal row label falls in [lo, hi) (stable compaction: count + scan + scatter)
__global__ void k_flag_range(const int32_t* __restrict__ lab, int64_t n, int32_t lo, int32_t hi,
                             uint32_t* __restrict__ flag) {
  for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < n;
       p += (int64_t)gridDim.x * blockDim.x)
    flag[p] = (lab[p] >= lo && lab[p] < hi) ? 1u : 0u;
}
__global__ void k_scatter_sel(const uint32_t* __restrict__ flag, const uint32_t* __restrict__ incl, int64_t n,
                              uint32_t* __restrict__ sel) {
  for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < n;
       p += (int64_t)gridDim.x * blockDim.x)
    if (flag[p]) sel[incl[p] - 1] = (uint32_t)p;
}
// out[s] = in[sel[s]] - shift
__global__ void k_gather_shift(const int32_t* __restrict__ in, const uint32_t* __restrict__ sel, int64_t n,
                               int32_t shift, int32_t* __restrict__ out) {
  for (int64_t s = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; s < n;
       s += (int64_t)gridDim.x * blockDim.x)
    out[s] = in[sel[s]] - shift;
}

struct RecArgs {
  const int32_t* idx[7];   // slot q source index array (canonical order)
  const int32_t* hmap[7] = {nullptr};  // slot q: factor row -> hot slot or -1 (null: no hot rows)
  int nslots;
  int recb;
  int pk = 0;              // packed 16-byte records (ModeStore::pk): slot q at bit sh[q]
  int sh[7] = {0};
  uint32_t hot[7] = {0};   // hot flag of slot q's field
  int rel = -1;            // slot stored as its row within the L2 block (blocks of blk rows)
  uint32_t blk = 1;
};

// rec[p] = {idx[q][perm[p]] ..., vals[perm[p]]}; a hot row is stored as 0x80000000 | hot slot
// (packed records: {sum_q field_q << sh[q], x}, field = row or hot[q] | hot slot)
__global__ void k_make_records(RecArgs a, const double* __restrict__ vals, const uint32_t* __restrict__ perm,
                               int64_t n, char* __restrict__ rec) {
  for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < n;
       p += (int64_t)gridDim.x * blockDim.x) {
    const uint32_t src = perm[p];
    char* r = rec + p * a.recb;
    if (a.pk) {
      unsigned long long key = 0;
      for (int q = 0; q < a.nslots; q++) {
        uint32_t v = (uint32_t)a.idx[q][src];
        if (q == a.rel) v %= a.blk;
        if (a.hmap[q]) {
          const int32_t h = a.hmap[q][v];
          if (h >= 0) v = a.hot[q] | (uint32_t)h;
        }
        key |= (unsigned long long)v << a.sh[q];
      }
      *reinterpret_cast<unsigned long long*>(r) = key;
      *reinterpret_cast<double*>(r + 8) = vals[src];
      continue;
    }
    int32_t* ri = reinterpret_cast<int32_t*>(r);
    for (int q = 0; q < a.nslots; q++) {
      int32_t v = a.idx[q][src];
      if (a.hmap[q]) {
        const int32_t h = a.hmap[q][v];
        if (h >= 0) v = (int32_t)(0x80000000u | (uint32_t)h);
      }
      ri[q] = v;
    }
    for (int q = a.nslots; q < (a.recb - 8) / 4; q++) ri[q] = 0;
    *reinterpret_cast<double*>(r + a.recb - 8) = vals[src];
  }
}

struct HotArgs {
  const int32_t* rows = nullptr;   // hot slot -> factor row (all factors, concatenated)
  int64_t off[7] = {0};            // slot q: first hot slot of its factor
  int pk = 0;                      // packed records: field q = (key >> sh[q]) & mask[q]
  int sh[7] = {0};
  uint32_t mask[7] = {0}, hot[7] = {0};
  int rel = -1;                    // block-relative slot: row = field + kb[p] * blk
  int64_t blk = 1;
  const int32_t* kb = nullptr;     // block of each record (L2-blocked copies)
};

// inverse of k_make_records for export: SoA arrays of the record slots + values
__global__ void k_split_records(const char* __restrict__ rec, int recb, int nslots, int64_t n, OutArgs out,
                                double* __restrict__ vals, HotArgs hot) {
  for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < n;
       p += (int64_t)gridDim.x * blockDim.x) {
    const char* r = rec + p * recb;
    if (hot.pk) {
      const unsigned long long key = *reinterpret_cast<const unsigned long long*>(r);
      for (int q = 0; q < nslots; q++) {
        uint32_t f = (uint32_t)(key >> hot.sh[q]) & hot.mask[q];
        int32_t v = (int32_t)f;
        if (f & hot.hot[q]) v = hot.rows[hot.off[q] + (f & ~hot.hot[q])];
        else if (q == hot.rel) v = (int32_t)(f + hot.kb[p] * hot.blk);
        out.idx[q][p] = v;
      }
      vals[p] = *reinterpret_cast<const double*>(r + 8);
      continue;
    }
    for (int q = 0; q < nslots; q++) {
      int32_t v = reinterpret_cast<const int32_t*>(r)[q];
      if (v < 0) v = hot.rows[hot.off[q] + (v & 0x7fffffff)];
      out.idx[q][p] = v;
    }
    vals[p] = *reinterpret_cast<const double*>(r + recb - 8);
  }
}

// rowptr[0] = 0, rowptr[i+1] = sum_{r<=i} counts[r]
cstf_status build_rowptr(const int32_t* d_key, int64_t n, int64_t I, DevBuf& rowptr, DevBuf& tmp,
                         cudaStream_t st) {
  CSTF_TRY(rowptr.alloc((size_t)(I + 1) * 8));
  DevBuf cnt;
  CSTF_TRY(cnt.alloc((size_t)I * 8));
  CSTF_CUDA(cudaMemsetAsync(cnt.p, 0, (size_t)I * 8, st));
  CSTF_CUDA(cudaMemsetAsync(rowptr.p, 0, 8, st));
  if (n > 0) {
    k_histogram<<<grid_for(n), kThreads, 0, st>>>(d_key, n, cnt.as<unsigned long long>());
    CSTF_LAUNCHED();
  }
  size_t tb = 0;
  CSTF_CUDA(cub::DeviceScan::InclusiveSum(nullptr, tb, cnt.as<unsigned long long>(),
                                          (unsigned long long*)(rowptr.as<int64_t>() + 1), I, st));
  CSTF_TRY(tmp.ensure(tb));
  CSTF_CUDA(cub::DeviceScan::InclusiveSum(tmp.p, tb, cnt.as<unsigned long long>(),
                                          (unsigned long long*)(rowptr.as<int64_t>() + 1), I, st));
  count_launch();
  CSTF_CUDA(cudaStreamSynchronize(st));  // cnt freed on return
  return CSTF_OK;
}

// L2-block decision for a mode copy with `nloc` nonzeros over `Iloc` output rows;
// Ioth[q] = rows of the factor gathered through record slot q (slots by increasing
// length).  Sets ms.tiled / blk_rows / nblk / tslot (L2 blocks, not SMEM slabs).
//  Default: block by the largest other factor t when it does not fit L2 even at
//  R = 32 (I_t * 256 B > L2) and the partial rows pay for themselves:
//   * short output mode, partial rows nearly free: nblk * I_n <= nnz / 64
//     (Delicious mode 4: 13.1 -> 10.3 ms), or
//   * long rows: >= 8 nonzeros per (row, block) on average, nnz >= 8 nblk I_n
//     (Amazon: 678 -> ~569 ms of MTTKRP per outer iteration).
//  Delicious modes 1-3 satisfy neither (blocking them measured slower).
//  CSTF_L2_BLOCK_ROWS / CSTF_L2_BLOCK_MAXROWS force it (tests, experiments).
// cov (optional, single GPU): per slot, the share of the nonzeros that fall on the
// factor's L2-capacity hottest rows (decide_hot).  When several other factors
// qualify, the one with the FLATTEST distribution (lowest share) is blocked and the
// skewed ones stream, since their hot rows are the ones a cache keeps (reading of
// VERDICT r01 "skew-aware blocking"; CSTF_L2_BLOCK_SKEW=0: always the longest).
// Packed 16-byte records (ModeStore::pk) for a copy with N-1 = 3 gathered slots (not an
// SMEM-slab copy), when the three fields fit 64 bits: field q holds values below
// max(I_q, hot slots of q) plus the hot flag bit if slot q has hot rows; in an L2-blocked
// copy the blocked slot holds the row within its block (pk_rel; Delicious mode 3: 61
// bits instead of 67, 10.60 -> 10.33 ms).  Halves the
// record stream of 4-mode tensors (Delicious modes 0 / 2: 60 / 58 bits; Enron: all
// modes).  Not for short-row copies (< 16 nonzeros per row): they are bound by
// instructions and latency, not bytes, and the decode costs more than the halved
// records save (Delicious mode 1: 11.25 -> 11.38 ms packed; modes 0 / 2: 9.40 -> 9.18,
// 9.44 -> 9.35 ms; Enron 7.75 -> 7.54 ms per outer iteration).  CSTF_PACK=0: never;
// CSTF_PACK=2: wherever the fields fit (tests).
void decide_pack(ModeStore& ms, int N, int64_t nloc, int64_t Iloc, const int64_t* Ioth, const int64_t* hotcnt) {
  ms.pk = false;
  ms.pk_rel = -1;
  const char* pe = getenv("CSTF_PACK");
  const int mode = pe ? atoi(pe) : 1;
  if (N != 4 || ms.slab || mode == 0) return;
  const int rel = ms.tiled ? ms.tslot : -1;     // L2 blocks: the blocked slot is block-relative
  if (mode != 2 && nloc < 16 * Iloc * (ms.tiled ? ms.nblk : 1)) return;
  int sh = 0;
  int shs[3];
  uint32_t masks[3], hots[3];
  for (int q = 0; q < 3; q++) {
    if (q == rel && hotcnt[q] > 0) return;      // (never: hot rows skip the blocked slot)
    const int64_t vmax = std::max<int64_t>(std::max<int64_t>(q == rel ? ms.blk_rows : Ioth[q], hotcnt[q]), 2) - 1;
    int b = 64 - __builtin_clzll((unsigned long long)vmax);
    const bool h = hotcnt[q] > 0;
    if (b + (h ? 1 : 0) > 32) return;
    hots[q] = h ? (1u << b) : 0u;
    b += h ? 1 : 0;
    masks[q] = b == 32 ? 0xffffffffu : ((1u << b) - 1u);
    shs[q] = sh;
    sh += b;
  }
  if (sh > 64) return;
  ms.pk = true;
  ms.pk_rel = rel;
  ms.recb = 16;
  for (int q = 0; q < 3; q++) { ms.pk_sh[q] = shs[q]; ms.pk_mask[q] = masks[q]; ms.pk_hot[q] = hots[q]; }
}

void set_pack_args(const ModeStore& ms, RecArgs& ra) {
  ra.recb = ms.recb;
  ra.pk = ms.pk ? 1 : 0;
  ra.rel = ms.pk_rel;
  ra.blk = ms.pk_rel >= 0 ? (uint32_t)ms.blk_rows : 1u;
  for (int q = 0; q < 7; q++) { ra.sh[q] = ms.pk_sh[q]; ra.hot[q] = ms.pk_hot[q]; }
}

void decide_l2_block(ModeStore& ms, int N, int64_t nloc, int64_t Iloc, const int64_t* Ioth,
                     const double* cov = nullptr) {
  if (N < 3 || (getenv("CSTF_L2_BLOCK") && atoi(getenv("CSTF_L2_BLOCK")) == 0)) return;
  const char* ov = getenv("CSTF_L2_BLOCK_ROWS");
  const bool forced = ov != nullptr;
  const int64_t l2rows = ov && atoll(ov) > 0 ? atoll(ov) : kL2Rows;
  const int64_t maxv = getenv("CSTF_L2_BLOCK_MAXROWS") ? atoll(getenv("CSTF_L2_BLOCK_MAXROWS"))
                                                      : ((int64_t)16 << 20);
  const bool skew = cov && !forced && !(getenv("CSTF_L2_BLOCK_SKEW") && atoi(getenv("CSTF_L2_BLOCK_SKEW")) == 0);
  int best = -1;
  // the longest other factor decides WHETHER the copy is blocked; with `skew`, a
  // flatter qualifying factor may then be blocked in its place
  for (int q = N - 2; q >= ((forced || skew) ? 0 : N - 2); q--) {     // largest other factor first
    const int64_t It = Ioth[q];
    const int64_t nb = (It + l2rows - 1) / l2rows;
    bool ok = It > 2 * l2rows && nb * Iloc < ((int64_t)1 << 31) && nloc >= 4 * nb * Iloc;
    if (forced)
      ok = ok && nb * Iloc <= maxv;
    else
      ok = ok && It * 256 > (int64_t)device_info().l2 && (nb * Iloc * 64 <= nloc || nloc >= 8 * nb * Iloc);
    if (!ok) {
      if (skew && q == N - 2) break;        // the longest does not qualify: not blocked
      continue;
    }
    if (!skew) { best = q; break; }
    if (best < 0 || cov[q] < cov[best]) best = q;
  }
  if (best >= 0) {
    const int64_t nb = (Ioth[best] + l2rows - 1) / l2rows;
    ms.tiled = true; ms.slab = false; ms.blk_rows = l2rows; ms.nblk = nb; ms.tslot = best;
  }
}

}  // namespace

// Partitioned copies: rows of every mode are dealt to
// ranks (cstf_partition_rows); all indices are relabelled to
// owner * B_n + local, and this rank keeps, for every mode n, the nonzeros whose
// mode-n row it owns, with the row index local to its block.
cstf_status decide_hot(cstf_tensor* X, DevBuf* c_idx, int64_t nout, DevBuf* hmap, double* cov, cudaStream_t st,
                       const int64_t* dims_override = nullptr);

cstf_status build_partitioned(cstf_tensor* X, DevBuf* c_idx, DevBuf& c_vals, int64_t nout, DevBuf& tmp,
                              cudaStream_t st) {
  const int N = X->N, P = X->nranks, rk = X->rank;
  DevBuf lab_idx[8];
  for (int n = 0; n < N; n++) {
    const int64_t I = X->dims[n];
    DevBuf cnt;
    CSTF_TRY(cnt.alloc((size_t)I * 8));
    CSTF_CUDA(cudaMemsetAsync(cnt.p, 0, (size_t)I * 8, st));
    if (nout) {
      k_histogram<<<grid_for(nout), kThreads, 0, st>>>(c_idx[n].as<int32_t>(), nout, cnt.as<unsigned long long>());
      CSTF_LAUNCHED();
    }
    std::vector<int64_t> counts((size_t)I), local((size_t)I);
    std::vector<int32_t> owner((size_t)I), lab((size_t)I);
    CSTF_CUDA(cudaMemcpyAsync(counts.data(), cnt.p, (size_t)I * 8, cudaMemcpyDeviceToHost, st));
    CSTF_CUDA(cudaStreamSynchronize(st));
    CSTF_TRY(cstf_partition_rows(I, counts.data(), P, owner.data(), local.data()));
    const int64_t B = (I + P - 1) / P;
    if ((int64_t)P * B >= ((int64_t)1 << 31)) return fail(CSTF_ERR_UNSUPPORTED, "padded mode length >= 2^31");
    X->rows_per_rank[n] = B;
    for (int64_t i = 0; i < I; i++) lab[(size_t)i] = (int32_t)(owner[(size_t)i] * B + local[(size_t)i]);
    CSTF_TRY(X->relabel[n].alloc((size_t)I * 4));
    CSTF_CUDA(cudaMemcpyAsync(X->relabel[n].p, lab.data(), (size_t)I * 4, cudaMemcpyHostToDevice, st));
    CSTF_TRY(lab_idx[n].alloc((size_t)nout * 4));
    if (nout) {
      k_map<<<grid_for(nout), kThreads, 0, st>>>(c_idx[n].as<int32_t>(), X->relabel[n].as<int32_t>(), nout,
                                                lab_idx[n].as<int32_t>());
      CSTF_LAUNCHED();
    }
    CSTF_CUDA(cudaStreamSynchronize(st));
  }
  // hot-row tables over the internal labels of the replicated factors (same rule as the
  // single-GPU store; every rank selects the same rows: the counts are global)
  DevBuf hmap[8];
  {
    double cov[8];
    int64_t Iint[8];
    for (int k = 0; k < N; k++) Iint[k] = (int64_t)P * X->rows_per_rank[k];
    static const bool kblock_env = getenv("CSTF_KBLOCK") && atoi(getenv("CSTF_KBLOCK")) > 0;
    if (!kblock_env) CSTF_TRY(decide_hot(X, lab_idx, nout, hmap, cov, st, Iint));
  }
  const int recb = record_bytes(N);
  for (int n = 0; n < N; n++) {
    ModeStore& ms = X->mode[n];
    const int64_t B = X->rows_per_rank[n];
    ms.I = B;
    ms.Ivirt = B;
    ms.tiled = false;
    ms.nblk = 1;
    ms.recb = recb;
    int k = 0;
    for (int m = 0; m < N; m++)
      if (m != n) ms.other[k++] = m;
    std::stable_sort(ms.other, ms.other + (N - 1), [&](int a, int b) { return X->dims[a] < X->dims[b]; });
    // select this rank's nonzeros of mode n (stable)
    DevBuf flag, incl, sel;
    int64_t ns = 0;
    CSTF_TRY(flag.alloc((size_t)nout * 4));
    CSTF_TRY(incl.alloc((size_t)nout * 4));
    if (nout) {
      k_flag_range<<<grid_for(nout), kThreads, 0, st>>>(lab_idx[n].as<int32_t>(), nout, (int32_t)(rk * B),
                                                        (int32_t)((rk + 1) * B), flag.as<uint32_t>());
      CSTF_LAUNCHED();
      size_t tb = 0;
      CSTF_CUDA(cub::DeviceScan::InclusiveSum(nullptr, tb, flag.as<uint32_t>(), incl.as<uint32_t>(), nout, st));
      CSTF_TRY(tmp.ensure(tb));
      CSTF_CUDA(cub::DeviceScan::InclusiveSum(tmp.p, tb, flag.as<uint32_t>(), incl.as<uint32_t>(), nout, st));
      count_launch();
      uint32_t last = 0;
      CSTF_CUDA(cudaMemcpyAsync(&last, incl.as<uint32_t>() + nout - 1, 4, cudaMemcpyDeviceToHost, st));
      CSTF_CUDA(cudaStreamSynchronize(st));
      ns = last;
    }
    CSTF_TRY(sel.alloc((size_t)ns * 4));
    if (nout) {
      k_scatter_sel<<<grid_for(nout), kThreads, 0, st>>>(flag.as<uint32_t>(), incl.as<uint32_t>(), nout,
                                                         sel.as<uint32_t>());
      CSTF_LAUNCHED();
    }
    // gathered keys: local row, then the other modes' internal labels by increasing length
    DevBuf kk[8], vv;
    for (int q = 0; q < N; q++) CSTF_TRY(kk[q].alloc((size_t)ns * 4));
    CSTF_TRY(vv.alloc((size_t)ns * 8));
    if (ns) {
      k_gather_shift<<<grid_for(ns), kThreads, 0, st>>>(lab_idx[n].as<int32_t>(), sel.as<uint32_t>(), ns,
                                                        (int32_t)(rk * B), kk[0].as<int32_t>());
      CSTF_LAUNCHED();
      for (int q = 0; q < N - 1; q++) {
        k_gather_shift<<<grid_for(ns), kThreads, 0, st>>>(lab_idx[ms.other[q]].as<int32_t>(), sel.as<uint32_t>(), ns, 0,
                                                          kk[q + 1].as<int32_t>());
        CSTF_LAUNCHED();
      }
      k_gather<double><<<grid_for(ns), kThreads, 0, st>>>(c_vals.as<double>(), sel.as<uint32_t>(), ns,
                                                          vv.as<double>());
      CSTF_LAUNCHED();
    }
    // L2 blocks over the internal labels of the largest other factor (local rows B)
    {
      int64_t Ioth[7];
      for (int q = 0; q < N - 1; q++) Ioth[q] = (int64_t)P * X->rows_per_rank[ms.other[q]];
      ms.slab = false;
      decide_l2_block(ms, N, ns, B, Ioth);
      ms.Ivirt = ms.nblk * B;
    }
    const int32_t* keys[9];
    int64_t kd[9];
    int nk = 0;
    DevBuf kbk, vrow;
    if (ms.tiled) {
      CSTF_TRY(kbk.alloc((size_t)ns * 4));
      CSTF_TRY(vrow.alloc((size_t)ns * 4));
      if (ns) {
        k_block_keys<<<grid_for(ns), kThreads, 0, st>>>(kk[ms.tslot + 1].as<int32_t>(), kk[0].as<int32_t>(), ns, B,
                                                        ms.blk_rows, kbk.as<int32_t>(), vrow.as<int32_t>());
        CSTF_LAUNCHED();
      }
      keys[nk] = kbk.as<int32_t>(); kd[nk++] = ms.nblk;
    }
    keys[nk] = kk[0].as<int32_t>();
    kd[nk++] = B;
    for (int q = 0; q < N - 1; q++) {
      keys[nk] = kk[q + 1].as<int32_t>();
      kd[nk++] = (int64_t)P * X->rows_per_rank[ms.other[q]];
    }
    DevBuf pm;
    CSTF_TRY(lsd_sort(keys, kd, nk, ns, pm, tmp, st));
    CSTF_TRY(build_rowptr(ms.tiled ? vrow.as<int32_t>() : kk[0].as<int32_t>(), ns, ms.Ivirt, ms.rowptr, tmp, st));
    ms.nnz = ns;
    RecArgs ra;
    ra.nslots = N - 1;
    for (int q = 0; q < N - 1; q++) ra.idx[q] = kk[q + 1].as<int32_t>();
    ms.hotmask = 0;
    {
      const bool slab_window = ms.tiled && ns / std::max<int64_t>(ms.nblk, 1) >= ((int64_t)16 << 20);
      for (int q = 0; q < N - 1 && !slab_window; q++)
        if (X->hot_cnt[ms.other[q]] > 0 && !(ms.tiled && q == ms.tslot)) {
          ra.hmap[q] = hmap[ms.other[q]].as<int32_t>();
          ms.hotmask |= 1 << q;
        }
    }
    {
      int64_t Ioth[7], hc[7];
      for (int q = 0; q < N - 1; q++) {
        Ioth[q] = (int64_t)P * X->rows_per_rank[ms.other[q]];
        hc[q] = (ms.hotmask & (1 << q)) ? X->hot_cnt[ms.other[q]] : 0;
      }
      decide_pack(ms, N, ns, B, Ioth, hc);
      set_pack_args(ms, ra);
    }
    CSTF_TRY(ms.rec.alloc((size_t)ns * ms.recb));
    if (ns) {
      k_make_records<<<grid_for(ns), kThreads, 0, st>>>(ra, vv.as<double>(), pm.as<uint32_t>(), ns, ms.rec.as<char>());
      CSTF_LAUNCHED();
    }
    CSTF_CUDA(cudaStreamSynchronize(st));
  }
  return CSTF_OK;
}

// Hot-row tables (single GPU).  A factor k whose
// rows do not fit half the L2 even at R = 32 (I_k * 256 B > L2 / 2) gets hot slots for
// its rows with the most nonzeros: at most half the device's persisting-L2 maximum
// in rows of 256 B (so the hot rows two factors contribute to one MTTKRP fit the
// set-aside), only rows with >= 2 nonzeros, ties by row index; slots are in
// descending count order.  CSTF_HOT=0 disables; CSTF_HOT_ROWS=<n> forces n hot rows
// per factor that has more than 2n rows (tests).  hmap[k] (device int32[I_k]) maps a
// row to its hot slot or -1 and is used while the mode copies are built.
// Also fills cov[k] (all factors larger than half the L2 at R = 32): the share of the
// nonzeros on the factor's L2-capacity hottest rows, for the skew-aware L2-block choice.
// dims_override (partitioned store): the internal (padded) factor lengths, c_idx the
// internal labels.
cstf_status decide_hot(cstf_tensor* X, DevBuf* c_idx, int64_t nout, DevBuf* hmap, double* cov, cudaStream_t st,
                       const int64_t* dims_override) {
  const int N = X->N;
  X->hot_total = 0;
  for (int k = 0; k < N; k++) cov[k] = 1.0;
  if (N < 3) return CSTF_OK;
  const bool hot_on = !(getenv("CSTF_HOT") && atoi(getenv("CSTF_HOT")) == 0);
  const char* fe = getenv("CSTF_HOT_ROWS");
  const int64_t forced = fe ? atoll(fe) : 0;
  int maxp = 0;
  cudaDeviceGetAttribute(&maxp, cudaDevAttrMaxPersistingL2CacheSize, device_info().device);
  const int64_t per_factor = !hot_on ? 0 : forced > 0 ? forced : (int64_t)maxp / 256 / 2;
  const int64_t l2rows = (int64_t)device_info().l2 / 256;
  std::vector<int32_t> all;
  for (int k = 0; k < N; k++) {
    X->hot_off[k] = (int64_t)all.size();
    X->hot_cnt[k] = 0;
    const int64_t I = dims_override ? dims_override[k] : X->dims[k];
    const bool big = forced > 0 ? I > 2 * forced : I * 256 > (int64_t)device_info().l2 / 2;
    if (!big || nout == 0) continue;
    DevBuf cnt;
    CSTF_TRY(cnt.alloc((size_t)I * 8));
    CSTF_CUDA(cudaMemsetAsync(cnt.p, 0, (size_t)I * 8, st));
    k_histogram<<<grid_for(nout), kThreads, 0, st>>>(c_idx[k].as<int32_t>(), nout, cnt.as<unsigned long long>());
    CSTF_LAUNCHED();
    std::vector<int64_t> counts((size_t)I);
    CSTF_CUDA(cudaMemcpyAsync(counts.data(), cnt.p, (size_t)I * 8, cudaMemcpyDeviceToHost, st));
    CSTF_CUDA(cudaStreamSynchronize(st));
    std::vector<int32_t> order((size_t)I);
    for (int64_t i = 0; i < I; i++) order[(size_t)i] = (int32_t)i;
    const int64_t H = std::min<int64_t>(per_factor, I);
    auto by_count = [&](int32_t a, int32_t b) { return counts[a] != counts[b] ? counts[a] > counts[b] : a < b; };
    {
      std::vector<int64_t> cs(counts);
      const int64_t C = std::min<int64_t>(l2rows, I);
      std::nth_element(cs.begin(), cs.begin() + (C - 1), cs.end(), std::greater<int64_t>());
      double top = 0.0;
      for (int64_t i = 0; i < C; i++) top += (double)cs[(size_t)i];
      cov[k] = top / (double)nout;
    }
    if (H < 1) continue;
    std::partial_sort(order.begin(), order.begin() + H, order.end(), by_count);
    int64_t h = 0;
    while (h < H && counts[(size_t)order[(size_t)h]] >= 2) h++;
    if (h == 0) continue;
    std::vector<int32_t> map((size_t)I, -1);
    for (int64_t s = 0; s < h; s++) map[(size_t)order[(size_t)s]] = (int32_t)s;
    CSTF_TRY(hmap[k].alloc((size_t)I * 4));
    CSTF_CUDA(cudaMemcpyAsync(hmap[k].p, map.data(), (size_t)I * 4, cudaMemcpyHostToDevice, st));
    CSTF_CUDA(cudaStreamSynchronize(st));
    all.insert(all.end(), order.begin(), order.begin() + h);
    X->hot_cnt[k] = h;
  }
  X->hot_total = (int64_t)all.size();
  if (X->hot_total) {
    CSTF_TRY(X->hot_rows.alloc(all.size() * 4));
    CSTF_CUDA(cudaMemcpyAsync(X->hot_rows.p, all.data(), all.size() * 4, cudaMemcpyHostToDevice, st));
    CSTF_CUDA(cudaStreamSynchronize(st));
  }
  return CSTF_OK;
}

cstf_status build_store(cstf_tensor* X, const int32_t* const* host_idx, const double* host_vals,
                        int64_t n, cudaStream_t st) {
  const int N = X->N;
  DevBuf tmp;  // cub temp storage
  // ---- 1. upload + validate
  DevBuf in_idx[8], in_vals;
  for (int m = 0; m < N; m++) {
    CSTF_TRY(in_idx[m].alloc((size_t)n * 4));
    if (n) CSTF_CUDA(cudaMemcpyAsync(in_idx[m].p, host_idx[m], (size_t)n * 4, cudaMemcpyHostToDevice, st));
  }
  CSTF_TRY(in_vals.alloc((size_t)n * 8));
  if (n) CSTF_CUDA(cudaMemcpyAsync(in_vals.p, host_vals, (size_t)n * 8, cudaMemcpyHostToDevice, st));
  {
    DevBuf bad;
    CSTF_TRY(bad.alloc(8));
    CSTF_CUDA(cudaMemsetAsync(bad.p, 0, 8, st));
    for (int m = 0; m < N && n > 0; m++) {
      k_count_invalid<<<grid_for(n), kThreads, 0, st>>>(in_idx[m].as<int32_t>(), n, X->dims[m],
                                                        bad.as<unsigned long long>());
      CSTF_LAUNCHED();
    }
    unsigned long long nbad = 0;
    CSTF_CUDA(cudaMemcpyAsync(&nbad, bad.p, 8, cudaMemcpyDeviceToHost, st));
    CSTF_CUDA(cudaStreamSynchronize(st));
    if (nbad) return fail(CSTF_ERR_INVALID_ARG, std::to_string(nbad) + " indices outside [0, dims[n])");
  }
  // ---- 2. canonical order: stable LSD radix sort by (i_1, ..., i_N)
  DevBuf perm_a;
  {
    const int32_t* keys[8];
    for (int m = 0; m < N; m++) keys[m] = in_idx[m].as<int32_t>();
    CSTF_TRY(lsd_sort(keys, X->dims, N, n, perm_a, tmp, st));
  }
  // ---- 3. gather into sorted order, free the inputs
  DevBuf s_idx[8], s_vals;
  for (int m = 0; m < N; m++) {
    CSTF_TRY(s_idx[m].alloc((size_t)n * 4));
    if (n) { k_gather<int32_t><<<grid_for(n), kThreads, 0, st>>>(in_idx[m].as<int32_t>(), perm_a.as<uint32_t>(), n, s_idx[m].as<int32_t>()); CSTF_LAUNCHED(); }
  }
  CSTF_TRY(s_vals.alloc((size_t)n * 8));
  if (n) { k_gather<double><<<grid_for(n), kThreads, 0, st>>>(in_vals.as<double>(), perm_a.as<uint32_t>(), n, s_vals.as<double>()); CSTF_LAUNCHED(); }
  CSTF_CUDA(cudaStreamSynchronize(st));
  for (int m = 0; m < N; m++) in_idx[m].release();
  in_vals.release();
  // ---- 4. duplicates: heads, segment ids, left-to-right sums
  IdxArgs sa;
  sa.N = N;
  for (int m = 0; m < N; m++) sa.idx[m] = s_idx[m].as<int32_t>();
  int64_t nout = 0;
  DevBuf c_idx[8], c_vals;
  {
    DevBuf head, segid;
    CSTF_TRY(head.alloc((size_t)n * 4));
    CSTF_TRY(segid.alloc((size_t)n * 4));
    if (n) {
      k_heads<<<grid_for(n), kThreads, 0, st>>>(sa, n, head.as<uint32_t>());
      CSTF_LAUNCHED();
      size_t tb = 0;
      CSTF_CUDA(cub::DeviceScan::InclusiveSum(nullptr, tb, head.as<uint32_t>(), segid.as<uint32_t>(), n, st));
      CSTF_TRY(tmp.ensure(tb));
      CSTF_CUDA(cub::DeviceScan::InclusiveSum(tmp.p, tb, head.as<uint32_t>(), segid.as<uint32_t>(), n, st));
      count_launch();
      uint32_t last = 0;
      CSTF_CUDA(cudaMemcpyAsync(&last, segid.as<uint32_t>() + n - 1, 4, cudaMemcpyDeviceToHost, st));
      CSTF_CUDA(cudaStreamSynchronize(st));
      nout = last;
    }
    // reuse perm_a as segment starts
    if (n) { k_seg_starts<<<grid_for(n), kThreads, 0, st>>>(head.as<uint32_t>(), segid.as<uint32_t>(), n, perm_a.as<uint32_t>()); CSTF_LAUNCHED(); }
    OutArgs oa;
    oa.N = N;
    for (int m = 0; m < N; m++) {
      CSTF_TRY(c_idx[m].alloc((size_t)nout * 4));
      oa.idx[m] = c_idx[m].as<int32_t>();
    }
    CSTF_TRY(c_vals.alloc((size_t)nout * 8));
    if (nout) {
      k_coalesce<<<grid_for(nout), kThreads, 0, st>>>(sa, s_vals.as<double>(), perm_a.as<uint32_t>(), nout, n, oa, c_vals.as<double>());
      CSTF_LAUNCHED();
    }
    CSTF_CUDA(cudaStreamSynchronize(st));
  }
  for (int m = 0; m < N; m++) s_idx[m].release();
  s_vals.release();
  perm_a.release();
  X->nnz = nout;
  // ---- 5. ||X||^2 and checksum (fixed grid => deterministic)
  {
    IdxArgs ca;
    ca.N = N;
    for (int m = 0; m < N; m++) ca.idx[m] = c_idx[m].as<int32_t>();
    DevBuf pn, ph, out;
    CSTF_TRY(pn.alloc(kFixedBlocks * 8));
    CSTF_TRY(ph.alloc(kFixedBlocks * 8));
    CSTF_TRY(out.alloc(16));
    k_norm_hash<<<kFixedBlocks, kThreads, 0, st>>>(ca, c_vals.as<double>(), nout, pn.as<double>(), ph.as<unsigned long long>());
    CSTF_LAUNCHED();
    k_norm_hash_final<<<1, 32, 0, st>>>(pn.as<double>(), ph.as<unsigned long long>(), kFixedBlocks, out.as<double>(), (unsigned long long*)(out.as<double>() + 1));
    CSTF_LAUNCHED();
    double hv[2];
    CSTF_CUDA(cudaMemcpyAsync(hv, out.p, 16, cudaMemcpyDeviceToHost, st));
    CSTF_CUDA(cudaStreamSynchronize(st));
    X->normX2 = hv[0];
    memcpy(&X->hash, &hv[1], 8);
  }
  if (X->partitioned) return build_partitioned(X, c_idx, c_vals, nout, tmp, st);
  // ---- 6. hot rows of the factors much larger than L2 (single GPU)
  DevBuf hmap[8];
  double cov[8];
  static const bool kblock_env = getenv("CSTF_KBLOCK") && atoi(getenv("CSTF_KBLOCK")) > 0;
  for (int k = 0; k < 8; k++) cov[k] = 1.0;
  if (!kblock_env) CSTF_TRY(decide_hot(X, c_idx, nout, hmap, cov, st));
  // ---- 7. per-mode copies: sorted by (i_n, other modes by increasing length), AoS records
  const int recb = record_bytes(N);
  for (int n_ = 0; n_ < N; n_++) {
    ModeStore& ms = X->mode[n_];
    ms.I = X->dims[n_];
    ms.nnz = nout;
    ms.recb = recb;
    int k = 0;
    for (int m = 0; m < N; m++)
      if (m != n_) ms.other[k++] = m;
    std::stable_sort(ms.other, ms.other + (N - 1), [&](int a, int b) { return X->dims[a] < X->dims[b]; });
    // Blocking decision (host logic).
    //  * L2 blocks (opt-in CSTF_L2_BLOCK_ROWS): block the largest other factor that does not fit
    //    in L2 (> 2 kL2Rows rows) into kL2Rows-row blocks, if the partial rows
    //    (nblk * I_n) stay within budget and average >= 4 nonzeros each, so the
    //    gathered slice of that factor stays L2-resident while its nonzeros stream.
    //  * SMEM slabs (opt-in CSTF_KBLOCK=1): kTileRows-row blocks of the longest
    //    other mode, staged in shared memory by the CTA.
    static const bool kblock_on = getenv("CSTF_KBLOCK") && atoi(getenv("CSTF_KBLOCK")) > 0;
    ms.tiled = false;
    ms.slab = false;
    ms.nblk = 1;
    int t = -1;
    if (N >= 3 && kblock_on) {
      t = ms.other[N - 2];
      const int64_t nb = (X->dims[t] + kTileRows - 1) / kTileRows;
      if (nb >= 2 && nb * ms.I <= ((int64_t)4 << 20) && nout >= 8 * nb * ms.I) {
        ms.tiled = ms.slab = true; ms.blk_rows = kTileRows; ms.nblk = nb; ms.tslot = N - 2;
      }
    } else {
      int64_t Ioth[7];
      double cq[7];
      for (int q = 0; q < N - 1; q++) { Ioth[q] = X->dims[ms.other[q]]; cq[q] = cov[ms.other[q]]; }
      decide_l2_block(ms, N, nout, ms.I, Ioth, cq);
      if (ms.tiled) t = ms.other[ms.tslot];
    }
    const int64_t nblk = ms.nblk;
    ms.Ivirt = ms.nblk * ms.I;
    const int32_t* keys[9];
    int64_t kd[9];
    int nk = 0;
    DevBuf kbk, vrow;
    if (ms.tiled) {
      CSTF_TRY(kbk.alloc((size_t)nout * 4));
      CSTF_TRY(vrow.alloc((size_t)nout * 4));
      k_block_keys<<<grid_for(nout), kThreads, 0, st>>>(c_idx[t].as<int32_t>(), c_idx[n_].as<int32_t>(), nout,
                                                        ms.I, ms.blk_rows, kbk.as<int32_t>(), vrow.as<int32_t>());
      CSTF_LAUNCHED();
      keys[nk] = kbk.as<int32_t>(); kd[nk++] = nblk;
    }
    keys[nk] = c_idx[n_].as<int32_t>();
    kd[nk++] = X->dims[n_];
    for (int q = 0; q < N - 1; q++) { keys[nk] = c_idx[ms.other[q]].as<int32_t>(); kd[nk++] = X->dims[ms.other[q]]; }
    DevBuf pm;
    CSTF_TRY(lsd_sort(keys, kd, nk, nout, pm, tmp, st));
    CSTF_TRY(build_rowptr(ms.tiled ? vrow.as<int32_t>() : c_idx[n_].as<int32_t>(), nout, ms.Ivirt, ms.rowptr, tmp, st));
    RecArgs ra;
    ra.nslots = N - 1;
    for (int q = 0; q < N - 1; q++) ra.idx[q] = c_idx[ms.other[q]].as<int32_t>();
    // hot rows in every slot of the copy except the L2-blocked one (its slab is
    // L2-resident by construction) and except copies whose blocks run under their own
    // persisting window (>= 16M nonzeros per block, mttkrp.cu)
    ms.hotmask = 0;
    const bool slab_window = ms.tiled && !ms.slab && nout / std::max<int64_t>(ms.nblk, 1) >= ((int64_t)16 << 20);
    for (int q = 0; q < N - 1 && !ms.slab && !slab_window; q++)
      if (X->hot_cnt[ms.other[q]] > 0 && !(ms.tiled && q == ms.tslot)) {
        ra.hmap[q] = hmap[ms.other[q]].as<int32_t>();
        ms.hotmask |= 1 << q;
      }
    {
      int64_t Ioth[7], hc[7];
      for (int q = 0; q < N - 1; q++) {
        Ioth[q] = X->dims[ms.other[q]];
        hc[q] = (ms.hotmask & (1 << q)) ? X->hot_cnt[ms.other[q]] : 0;
      }
      decide_pack(ms, N, nout, ms.I, Ioth, hc);
      set_pack_args(ms, ra);
    }
    CSTF_TRY(ms.rec.alloc((size_t)nout * ms.recb));
    if (nout) {
      k_make_records<<<grid_for(nout), kThreads, 0, st>>>(ra, c_vals.as<double>(), pm.as<uint32_t>(), nout,
                                                          ms.rec.as<char>());
      CSTF_LAUNCHED();
    }
    CSTF_CUDA(cudaStreamSynchronize(st));
  }
  return CSTF_OK;
}

// Canonical order back from the mode-0 copy: expand rows, split the records,
// stable sort by (i_1..i_N), copy to the host.
cstf_status export_store(const cstf_tensor* X, int32_t* const* host_idx, double* host_vals) {
  const ModeStore& ms = X->mode[0];
  const int N = X->N;
  const int64_t n = ms.nnz;
  cudaStream_t st = 0;
  if (n == 0) return CSTF_OK;
  DevBuf soa[8], vals, tmp, perm, out;
  for (int m = 0; m < N; m++) CSTF_TRY(soa[m].alloc((size_t)n * 4));
  CSTF_TRY(vals.alloc((size_t)n * 8));
  DevBuf kbv;
  if (ms.pk_rel >= 0) CSTF_TRY(kbv.alloc((size_t)n * 4));
  k_expand_rows<<<grid_for(ms.Ivirt), kThreads, 0, st>>>(ms.rowptr.as<int64_t>(), ms.Ivirt, ms.I,
                                                          soa[0].as<int32_t>(),
                                                          ms.pk_rel >= 0 ? kbv.as<int32_t>() : nullptr);
  CSTF_LAUNCHED();
  OutArgs oa;
  oa.N = N - 1;
  for (int q = 0; q < N - 1; q++) oa.idx[q] = soa[ms.other[q]].as<int32_t>();
  HotArgs ha;
  ha.rows = X->hot_rows.as<int32_t>();
  for (int q = 0; q < N - 1; q++) ha.off[q] = X->hot_off[ms.other[q]];
  ha.pk = ms.pk ? 1 : 0;
  for (int q = 0; q < 7; q++) { ha.sh[q] = ms.pk_sh[q]; ha.mask[q] = ms.pk_mask[q]; ha.hot[q] = ms.pk_hot[q]; }
  ha.rel = ms.pk_rel;
  ha.blk = ms.blk_rows;
  ha.kb = ms.pk_rel >= 0 ? kbv.as<int32_t>() : nullptr;
  k_split_records<<<grid_for(n), kThreads, 0, st>>>(ms.rec.as<char>(), ms.recb, N - 1, n, oa, vals.as<double>(), ha);
  CSTF_LAUNCHED();
  const int32_t* keys[8];
  for (int m = 0; m < N; m++) keys[m] = soa[m].as<int32_t>();
  CSTF_TRY(lsd_sort(keys, X->dims, N, n, perm, tmp, st));
  CSTF_TRY(out.alloc((size_t)n * 8));
  for (int m = 0; m < N; m++) {
    k_gather<int32_t><<<grid_for(n), kThreads, 0, st>>>(soa[m].as<int32_t>(), perm.as<uint32_t>(), n, out.as<int32_t>());
    CSTF_LAUNCHED();
    CSTF_CUDA(cudaMemcpy(host_idx[m], out.p, (size_t)n * 4, cudaMemcpyDeviceToHost));
  }
  k_gather<double><<<grid_for(n), kThreads, 0, st>>>(vals.as<double>(), perm.as<uint32_t>(), n, out.as<double>());
  CSTF_LAUNCHED();
  CSTF_CUDA(cudaMemcpy(host_vals, out.p, (size_t)n * 8, cudaMemcpyDeviceToHost));
  return CSTF_OK;
}

}  // namespace cstf
