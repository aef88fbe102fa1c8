// Gather-path probe for the MTTKRP access pattern (tools only, not the product):
// 16 lanes x 16 B cover one 256 B factor row (R = 32 FP64); a warp gathers the
// rows of two nonzeros per load instruction, two tables (the two other modes).
// Variants: cache policy of the row loads (default / L1::no_allocate / .cg L2-only /
// L1::evict_last) and table size (L1-resident, L2-resident, HBM).
#include <cstdio>
#include <cstdint>
#include <vector>
#include <cuda_runtime.h>
#define CK(x) do{cudaError_t e=(x); if(e!=cudaSuccess){printf("CUDA %s @%d\n",cudaGetErrorString(e),__LINE__); return 1;}}while(0)

template <int POL>
__device__ __forceinline__ double2 ld16(const double* p) {
  double2 v;
  if (POL == 0) v = __ldg(reinterpret_cast<const double2*>(p));
  else if (POL == 1)
    asm volatile("ld.global.nc.L1::no_allocate.v2.f64 {%0,%1}, [%2];" : "=d"(v.x), "=d"(v.y) : "l"(p));
  else if (POL == 2)
    asm volatile("ld.global.cg.v2.f64 {%0,%1}, [%2];" : "=d"(v.x), "=d"(v.y) : "l"(p));
  else
    asm volatile("ld.global.nc.L1::evict_last.v2.f64 {%0,%1}, [%2];" : "=d"(v.x), "=d"(v.y) : "l"(p));
  return v;
}

template <int POL>
__global__ void __launch_bounds__(256) gather16(const double* __restrict__ B, const double* __restrict__ C,
    const int2* __restrict__ jk, int64_t nnz, double* out) {
  const int lane = threadIdx.x & 31, grp = lane >> 4, gl = lane & 15;
  int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  int64_t nw = (gridDim.x * (int64_t)blockDim.x) >> 5;
  double a0 = 0, a1 = 0;
  for (int64_t p0 = warp * 32; p0 < nnz; p0 += nw * 32) {
    const int2 r = jk[p0 + lane];
#pragma unroll 4
    for (int q = 0; q < 16; q++) {
      const int src = 2 * q + grp;
      const int j = __shfl_sync(0xffffffffu, r.x, src), k = __shfl_sync(0xffffffffu, r.y, src);
      const double2 b = ld16<POL>(B + (size_t)j * 32 + 2 * gl);
      const double2 c = ld16<POL>(C + (size_t)k * 32 + 2 * gl);
      a0 = fma(b.x, c.x, a0);
      a1 = fma(b.y, c.y, a1);
    }
  }
  out[blockIdx.x * (int64_t)blockDim.x + threadIdx.x] = a0 + a1;
}

template <int POL>
int run(const char* name, const double* B, const double* C, const int2* jk, int64_t nnz, double* out, int sms,
        long long rows) {
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1); float ms;
  for (int bpsm : {4, 8}) {
    const int grid = sms * bpsm;
    gather16<POL><<<grid, 256>>>(B, C, jk, nnz, out);
    cudaEventRecord(e0);
    gather16<POL><<<grid, 256>>>(B, C, jk, nnz, out);
    cudaEventRecord(e1);
    CK(cudaEventSynchronize(e1));
    cudaEventElapsedTime(&ms, e0, e1);
    printf("%-14s rows=%-9lld bpsm%d: %.3f ms  %.2f Gnnz/s  gathered %.0f GB/s\n", name, rows, bpsm, ms,
           nnz / ms / 1e6, nnz * 512.0 / ms / 1e6);
  }
  return 0;
}

int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  double* out; CK(cudaMalloc(&out, 64 << 20));
  const int64_t nnz = 64 << 20;
  int2* jk; CK(cudaMalloc(&jk, nnz * 8));
  std::vector<int2> h(nnz);
  for (long long rows : {200LL, 9000LL, 29000LL, 2500000LL}) {
    double *B, *C;
    CK(cudaMalloc(&B, rows * 256)); CK(cudaMalloc(&C, rows * 256));
    cudaMemset(B, 0, rows * 256); cudaMemset(C, 0, rows * 256);
    uint64_t s = 12345;
    for (int64_t i = 0; i < nnz; i++) {
      s = s * 6364136223846793005ULL + 1442695040888963407ULL; h[i].x = (int)((s >> 33) % rows);
      s = s * 6364136223846793005ULL + 1442695040888963407ULL; h[i].y = (int)((s >> 33) % rows);
    }
    cudaMemcpy(jk, h.data(), nnz * 8, cudaMemcpyHostToDevice);
    run<0>("default", B, C, jk, nnz, out, sms, rows);
    run<1>("no_allocate", B, C, jk, nnz, out, sms, rows);
    run<2>("cg", B, C, jk, nnz, out, sms, rows);
    run<3>("evict_last", B, C, jk, nnz, out, sms, rows);
    cudaFree(B); cudaFree(C);
  }
  return 0;
}
