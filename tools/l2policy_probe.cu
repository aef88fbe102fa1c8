// L2 eviction-priority probe (tools only): power-law gathers of 256-byte rows from
// tables much larger than L2 (Delicious-shaped: 17.3M rows gamma=2 and 2.5M rows
// gamma=3), with the hot rows first (row id = rank).  Compares plain loads with
// loads that tag rows id < H_k evict_last and the rest evict_first.
#include <algorithm>
#include <cstdio>
#include <cstdint>
#include <cmath>
#include <vector>
#include <cuda_runtime.h>
#define CK(x) do{cudaError_t e=(x); if(e!=cudaSuccess){printf("CUDA %s @%d\n",cudaGetErrorString(e),__LINE__); return 1;}}while(0)

__device__ __forceinline__ double2 ld_pol(const double* p, uint64_t pol) {
  double2 v;
  asm volatile("ld.global.nc.L2::cache_hint.v2.f64 {%0,%1}, [%2], %3;" : "=d"(v.x), "=d"(v.y) : "l"(p), "l"(pol));
  return v;
}

template <int MODE>   // 0 plain; 1 last/first; 2 normal for all; 3 last/normal; 4 last/unchanged
__global__ void __launch_bounds__(256) gather(const double* __restrict__ B, const double* __restrict__ C,
    const int2* __restrict__ jk, int64_t nnz, int hB, int hC, double* out) {
  const int lane = threadIdx.x & 31, grp = lane >> 4, gl = lane & 15;
  int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  int64_t nw = (gridDim.x * (int64_t)blockDim.x) >> 5;
  uint64_t pl = 0, pf = 0;
  if (MODE == 1 || MODE == 3 || MODE == 4)
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pl));
  if (MODE == 1) asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pf));
  if (MODE == 2 || MODE == 3) asm volatile("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(pf));
  if (MODE == 2) pl = pf;
  if (MODE == 4) asm volatile("createpolicy.fractional.L2::evict_unchanged.b64 %0, 1.0;" : "=l"(pf));
  double a0 = 0, a1 = 0;
  for (int64_t p0 = warp * 32; p0 < nnz; p0 += nw * 32) {
    const int2 r = jk[p0 + lane];
#pragma unroll 4
    for (int q = 0; q < 16; q++) {
      const int src = 2 * q + grp;
      const int j = __shfl_sync(0xffffffffu, r.x, src), k = __shfl_sync(0xffffffffu, r.y, src);
      double2 b, c;
      if (MODE == 0) {
        b = __ldg(reinterpret_cast<const double2*>(B + (size_t)j * 32 + 2 * gl));
        c = __ldg(reinterpret_cast<const double2*>(C + (size_t)k * 32 + 2 * gl));
      } else {
        b = ld_pol(B + (size_t)j * 32 + 2 * gl, j < hB ? pl : pf);
        c = ld_pol(C + (size_t)k * 32 + 2 * gl, k < hC ? pl : pf);
      }
      a0 = fma(b.x, c.x, a0);
      a1 = fma(b.y, c.y, a1);
    }
  }
  out[blockIdx.x * (int64_t)blockDim.x + threadIdx.x] = a0 + a1;
}

int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  double* out; CK(cudaMalloc(&out, 64 << 20));
  const int64_t nnz = 140000000;
  const int64_t IB = 17300000, IC = 2500000;
  int2* jk; CK(cudaMalloc(&jk, nnz * 8));
  std::vector<int2> h(nnz);
  uint64_t s = 777;
  auto u = [&]() { s = s * 6364136223846793005ULL + 1442695040888963407ULL; return ((s >> 11) + 0.5) / 9007199254740992.0; };
  for (int64_t i = 0; i < nnz; i++) {
    h[i].x = (int)std::min<int64_t>((int64_t)(IB * std::pow(u(), 2.0)), IB - 1);
    h[i].y = (int)std::min<int64_t>((int64_t)(IC * std::pow(u(), 3.0)), IC - 1);
  }
  CK(cudaMemcpy(jk, h.data(), nnz * 8, cudaMemcpyHostToDevice));
  double *B, *C;
  CK(cudaMalloc(&B, IB * 256)); CK(cudaMalloc(&C, IC * 256));
  cudaMemset(B, 0, IB * 256); cudaMemset(C, 0, IC * 256);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1); float ms;
  const int grid = sms * 8;
  gather<0><<<grid, 256>>>(B, C, jk, nnz, 0, 0, out);
  cudaEventRecord(e0); gather<0><<<grid, 256>>>(B, C, jk, nnz, 0, 0, out); cudaEventRecord(e1);
  CK(cudaEventSynchronize(e1)); cudaEventElapsedTime(&ms, e0, e1);
  printf("plain                      : %.3f ms\n", ms);
  // hot budgets in rows (256 B each): split between the two tables
  const int hbs[][2] = {{0, 200000}, {0, 400000}, {50000, 300000}, {200000, 200000}};
#define RUN(MD)                                                                                     \
  for (auto& hb : hbs) {                                                                            \
    gather<MD><<<grid, 256>>>(B, C, jk, nnz, hb[0], hb[1], out);                                    \
    cudaEventRecord(e0); gather<MD><<<grid, 256>>>(B, C, jk, nnz, hb[0], hb[1], out); cudaEventRecord(e1); \
    CK(cudaEventSynchronize(e1)); cudaEventElapsedTime(&ms, e0, e1);                                \
    printf("mode %d hB=%7d hC=%7d (%5.1f MB): %.3f ms\n", MD, hb[0], hb[1], (hb[0] + hb[1]) * 256.0 / 1e6, ms); \
  }
  RUN(1) RUN(2) RUN(3) RUN(4)
  // persisting-L2 set-aside + access-policy window over the hottest rows of one table
  cudaDeviceProp prop; cudaGetDeviceProperties(&prop, 0);
  printf("persistingL2CacheMaxSize %d MB, accessPolicyMaxWindowSize %d MB\n", prop.persistingL2CacheMaxSize >> 20,
         prop.accessPolicyMaxWindowSize >> 20);
  cudaStream_t st; cudaStreamCreate(&st);
  for (double frac : {0.25, 0.5, 0.75}) {
    size_t setaside = (size_t)(prop.persistingL2CacheMaxSize * frac);
    CK(cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, setaside));
    for (int which = 0; which < 2; which++) {
      for (double mult : {0.5, 1.0, 2.0}) {
        cudaStreamAttrValue v = {};
        size_t bytes = (size_t)(setaside * mult);
        if (bytes > (size_t)prop.accessPolicyMaxWindowSize) bytes = prop.accessPolicyMaxWindowSize;
        v.accessPolicyWindow.base_ptr = which ? (void*)B : (void*)C;
        v.accessPolicyWindow.num_bytes = bytes;
        v.accessPolicyWindow.hitRatio = (float)std::min(1.0, (double)setaside / bytes);
        v.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
        v.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
        CK(cudaStreamSetAttribute(st, cudaStreamAttributeAccessPolicyWindow, &v));
        gather<0><<<grid, 256, 0, st>>>(B, C, jk, nnz, 0, 0, out);
        cudaEventRecord(e0, st); gather<0><<<grid, 256, 0, st>>>(B, C, jk, nnz, 0, 0, out); cudaEventRecord(e1, st);
        CK(cudaEventSynchronize(e1)); cudaEventElapsedTime(&ms, e0, e1);
        printf("window on %s: setaside %.0f MB, window %.0f MB: %.3f ms\n", which ? "B(17.3M,g2)" : "C(2.5M,g3)",
               setaside / 1e6, bytes / 1e6, ms);
        v.accessPolicyWindow.num_bytes = 0;
        cudaStreamSetAttribute(st, cudaStreamAttributeAccessPolicyWindow, &v);
        cudaCtxResetPersistingL2Cache();
      }
    }
  }
  return 0;
}
