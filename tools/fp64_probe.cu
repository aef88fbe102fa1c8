// FP64 pipe probe (tools only): do DMMA and DFMA share one datapath on sm_100a?
// Throughput of DMMA alone, DFMA alone, and both interleaved in one warp; also
// the larger f64 mma shapes (m16n8k4 / m16n8k8 / m16n8k16).
#include <cstdio>
#include <cuda_runtime.h>
#define CK(x) do{cudaError_t e=(x); if(e!=cudaSuccess){printf("CUDA %s @%d\n",cudaGetErrorString(e),__LINE__); return 1;}}while(0)

template <int NMMA, int NFMA>
__global__ void mix(double* out, int iters) {
  double a = threadIdx.x * 1e-3, b = threadIdx.x * 2e-3;
  double c[8][2];
  double x[16];
#pragma unroll
  for (int t = 0; t < 8; t++) { c[t][0] = 0; c[t][1] = 0; }
#pragma unroll
  for (int t = 0; t < 16; t++) x[t] = threadIdx.x + t;
  for (int i = 0; i < iters; i++) {
#pragma unroll
    for (int t = 0; t < NMMA; t++)
      asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
                   : "+d"(c[t & 7][0]), "+d"(c[t & 7][1]) : "d"(a), "d"(b));
#pragma unroll
    for (int t = 0; t < NFMA; t++) x[t & 15] = fma(x[t & 15], a, 0.5);
  }
  double s = 0;
#pragma unroll
  for (int t = 0; t < 8; t++) s += c[t][0] + c[t][1];
#pragma unroll
  for (int t = 0; t < 16; t++) s += x[t];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

template <int K>
__global__ void big(double* out, int iters) {
  double a[K / 2 > 0 ? K / 2 : 1], b[K / 4 > 0 ? K / 4 : 1];
#pragma unroll
  for (int t = 0; t < (K / 2 > 0 ? K / 2 : 1); t++) a[t] = threadIdx.x * 1e-3 + t;
#pragma unroll
  for (int t = 0; t < (K / 4 > 0 ? K / 4 : 1); t++) b[t] = threadIdx.x * 2e-3 + t;
  double c[8][4];
#pragma unroll
  for (int t = 0; t < 8; t++) for (int u = 0; u < 4; u++) c[t][u] = 0;
  for (int i = 0; i < iters; i++) {
#pragma unroll
    for (int t = 0; t < 8; t++) {
      if (K == 4)
        asm volatile("mma.sync.aligned.m16n8k4.row.col.f64.f64.f64.f64 {%0,%1,%2,%3}, {%4,%5}, {%6}, {%0,%1,%2,%3};\n"
                     : "+d"(c[t][0]), "+d"(c[t][1]), "+d"(c[t][2]), "+d"(c[t][3]) : "d"(a[0]), "d"(a[1]), "d"(b[0]));
      else if (K == 8)
        asm volatile("mma.sync.aligned.m16n8k8.row.col.f64.f64.f64.f64 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, {%0,%1,%2,%3};\n"
                     : "+d"(c[t][0]), "+d"(c[t][1]), "+d"(c[t][2]), "+d"(c[t][3])
                     : "d"(a[0]), "d"(a[1]), "d"(a[2]), "d"(a[3]), "d"(b[0]), "d"(b[1]));
      else
        asm volatile("mma.sync.aligned.m16n8k16.row.col.f64.f64.f64.f64 {%0,%1,%2,%3}, {%4,%5,%6,%7,%8,%9,%10,%11}, {%12,%13,%14,%15}, {%0,%1,%2,%3};\n"
                     : "+d"(c[t][0]), "+d"(c[t][1]), "+d"(c[t][2]), "+d"(c[t][3])
                     : "d"(a[0]), "d"(a[1]), "d"(a[2]), "d"(a[3]), "d"(a[4]), "d"(a[5]), "d"(a[6]), "d"(a[7]),
                       "d"(b[0]), "d"(b[1]), "d"(b[2]), "d"(b[3]));
    }
  }
  double s = 0;
#pragma unroll
  for (int t = 0; t < 8; t++) for (int u = 0; u < 4; u++) s += c[t][u];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

template <int NMMA, int NFMA>
void runmix(double* out, int sms) {
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1); float ms;
  const int grid = sms * 4, bs = 256, iters = 4000;
  mix<NMMA, NFMA><<<grid, bs>>>(out, 10);
  cudaEventRecord(e0); mix<NMMA, NFMA><<<grid, bs>>>(out, iters); cudaEventRecord(e1);
  cudaEventSynchronize(e1); cudaEventElapsedTime(&ms, e0, e1);
  const double warps = (double)grid * bs / 32 * iters;
  const double fm = warps * NMMA * 2 * 256, ff = warps * NFMA * 2 * 32;
  printf("mix dmma%-2d dfma%-2d: %.3f ms  dmma %.2f TF  dfma %.2f TF  total %.2f TF\n", NMMA, NFMA, ms,
         fm / ms / 1e9, ff / ms / 1e9, (fm + ff) / ms / 1e9);
}

template <int K>
void runbig(double* out, int sms) {
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1); float ms;
  const int grid = sms * 4, bs = 256, iters = 2000;
  big<K><<<grid, bs>>>(out, 10);
  cudaEventRecord(e0); big<K><<<grid, bs>>>(out, iters); cudaEventRecord(e1);
  cudaEventSynchronize(e1); cudaEventElapsedTime(&ms, e0, e1);
  const double warps = (double)grid * bs / 32 * iters;
  printf("m16n8k%-2d: %.3f ms  %.2f TF\n", K, ms, warps * 8 * 2.0 * 16 * 8 * K / ms / 1e9);
}

// latency: one warp per SM (or W warps), NCH independent accumulator chains
template <int NCH>
__global__ void lat(double* out, int iters, long long* cyc) {
  double a = threadIdx.x * 1e-3, b = threadIdx.x * 2e-3;
  double c[NCH][2];
#pragma unroll
  for (int t = 0; t < NCH; t++) { c[t][0] = 0; c[t][1] = 0; }
  long long t0 = clock64();
  for (int i = 0; i < iters; i++) {
#pragma unroll
    for (int t = 0; t < NCH; t++)
      asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
                   : "+d"(c[t][0]), "+d"(c[t][1]) : "d"(a), "d"(b));
  }
  long long t1 = clock64();
  double s = 0;
#pragma unroll
  for (int t = 0; t < NCH; t++) s += c[t][0] + c[t][1];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
  if (threadIdx.x == 0 && blockIdx.x == 0) *cyc = t1 - t0;
}

template <int NCH>
void runlat(double* out, long long* dc, int warps) {
  const int iters = 2000;
  lat<NCH><<<1, 32 * warps>>>(out, 10, dc);
  lat<NCH><<<1, 32 * warps>>>(out, iters, dc);
  long long c = 0;
  cudaMemcpy(&c, dc, 8, cudaMemcpyDeviceToHost);
  printf("DMMA chains %d warps/CTA %2d: %.1f cycles per DMMA per warp-chain step (%.2f cycles per DMMA issued)\n",
         NCH, warps, (double)c / iters, (double)c / iters / NCH / warps);
}

int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  double* out; CK(cudaMalloc(&out, 64 << 20));
  runmix<8, 0>(out, sms);
  runmix<0, 16>(out, sms);
  runmix<8, 4>(out, sms);
  runmix<8, 8>(out, sms);
  runmix<8, 16>(out, sms);
  runmix<8, 32>(out, sms);
  long long* dc; cudaMalloc(&dc, 8);
  runlat<1>(out, dc, 1); runlat<2>(out, dc, 1); runlat<4>(out, dc, 1); runlat<8>(out, dc, 1);
  runlat<4>(out, dc, 4); runlat<4>(out, dc, 8); runlat<4>(out, dc, 12); runlat<8>(out, dc, 4); runlat<8>(out, dc, 8);
  runbig<4>(out, sms);
  runbig<8>(out, sms);
  runbig<16>(out, sms);
  CK(cudaDeviceSynchronize());
  return 0;
}
