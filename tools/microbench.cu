// Microbenchmarks that set the B200 design numbers for the cSTF path:
// FP64 DFMA peak, FP64 DMMA (mma.sync m8n8k4 f64) peak, L2/HBM random-row
// gather bandwidth for 256 B factor rows (the MTTKRP access), HBM stream.
#include <cstdio>
#include <cstdint>
#include <vector>
#include <cuda_runtime.h>
#define CK(x) do{cudaError_t e=(x); if(e!=cudaSuccess){printf("CUDA %s @%d\n",cudaGetErrorString(e),__LINE__); return 1;}}while(0)

__global__ void dfma_kernel(double* out, int iters, double a) {
  double x0=threadIdx.x, x1=x0+1, x2=x0+2, x3=x0+3, x4=x0+4, x5=x0+5, x6=x0+6, x7=x0+7;
  for (int i=0;i<iters;i++){
#pragma unroll
    for(int j=0;j<8;j++){
      x0=fma(x0,a,0.5); x1=fma(x1,a,0.5); x2=fma(x2,a,0.5); x3=fma(x3,a,0.5);
      x4=fma(x4,a,0.5); x5=fma(x5,a,0.5); x6=fma(x6,a,0.5); x7=fma(x7,a,0.5);
    }
  }
  out[blockIdx.x*blockDim.x+threadIdx.x]=x0+x1+x2+x3+x4+x5+x6+x7;
}

__global__ void dmma_kernel(double* out, int iters) {
  double a = threadIdx.x*1e-3, b = threadIdx.x*2e-3;
  double c[8][2];
#pragma unroll
  for(int t=0;t<8;t++){c[t][0]=0;c[t][1]=0;}
  for(int i=0;i<iters;i++){
#pragma unroll
    for(int t=0;t<8;t++){
      asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
        : "+d"(c[t][0]), "+d"(c[t][1]) : "d"(a), "d"(b));
    }
  }
  double s=0;
#pragma unroll
  for(int t=0;t<8;t++) s+=c[t][0]+c[t][1];
  out[blockIdx.x*blockDim.x+threadIdx.x]=s;
}

// warp per nnz stream; lane = column (R=32); gather rows of B and C.
__global__ void gather_kernel(const double* __restrict__ B, const double* __restrict__ C,
    const int* __restrict__ jj, const int* __restrict__ kk, int64_t nnz, double* out) {
  int lane = threadIdx.x & 31;
  int64_t warp = (blockIdx.x*(int64_t)blockDim.x + threadIdx.x) >> 5;
  int64_t nw = (gridDim.x*(int64_t)blockDim.x) >> 5;
  double acc = 0;
  for (int64_t p0 = warp*32; p0 < nnz; p0 += nw*32) {
    int j = jj[p0+lane], k = kk[p0+lane];
#pragma unroll 8
    for (int q=0;q<32;q++){
      int jq = __shfl_sync(0xffffffff, j, q), kq = __shfl_sync(0xffffffff, k, q);
      acc += __ldg(B + (int64_t)jq*32 + lane) * __ldg(C + (int64_t)kq*32 + lane);
    }
  }
  out[blockIdx.x*blockDim.x+threadIdx.x] = acc;
}

__global__ void copy_kernel(const double2* __restrict__ a, double2* __restrict__ b, int64_t n) {
  for (int64_t i = blockIdx.x*(int64_t)blockDim.x+threadIdx.x; i<n; i+= (int64_t)gridDim.x*blockDim.x) b[i]=a[i];
}

int main(){
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  int l2; cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, 0);
  printf("SMs %d L2 %d\n", sms, l2);
  double* out; CK(cudaMalloc(&out, 64<<20));
  cudaEvent_t e0,e1; cudaEventCreate(&e0); cudaEventCreate(&e1); float ms;
  // DFMA
  for (int bs : {256, 512}) for (int bpsm : {2,4,8}) {
    int grid = sms*bpsm, iters=4000;
    dfma_kernel<<<grid,bs>>>(out, 10, 1.0000001);
    cudaEventRecord(e0); dfma_kernel<<<grid,bs>>>(out, iters, 1.0000001); cudaEventRecord(e1); CK(cudaEventSynchronize(e1));
    cudaEventElapsedTime(&ms,e0,e1);
    double fl = 2.0*64*iters*(double)grid*bs; printf("DFMA bs%d bpsm%d: %.2f TFLOP/s\n", bs,bpsm, fl/ms/1e9);
  }
  for (int bs : {128, 256, 512}) for (int bpsm : {2,4,8}) {
    int grid = sms*bpsm, iters=4000;
    dmma_kernel<<<grid,bs>>>(out, 10);
    cudaEventRecord(e0); dmma_kernel<<<grid,bs>>>(out, iters); cudaEventRecord(e1); CK(cudaEventSynchronize(e1));
    cudaEventElapsedTime(&ms,e0,e1);
    double fl = 2.0*256*8*iters*(double)grid*(bs/32); printf("DMMA bs%d bpsm%d: %.2f TFLOP/s\n", bs,bpsm, fl/ms/1e9);
  }
  // gather
  int64_t nnz = 64<<20;
  int *jj,*kk; CK(cudaMalloc(&jj,nnz*4)); CK(cudaMalloc(&kk,nnz*4));
  std::vector<int> h(nnz);
  for (int64_t rows : {8192LL, 29000LL, 131072LL, 1000000LL, 17300000LL}) {
    double *B,*C; CK(cudaMalloc(&B, rows*256)); CK(cudaMalloc(&C, rows*256));
    cudaMemset(B,0,rows*256); cudaMemset(C,0,rows*256);
    uint64_t s=12345;
    for (int64_t i=0;i<nnz;i++){ s=s*6364136223846793005ULL+1442695040888963407ULL; h[i]=(int)((s>>33)%rows);} cudaMemcpy(jj,h.data(),nnz*4,cudaMemcpyHostToDevice);
    for (int64_t i=0;i<nnz;i++){ s=s*6364136223846793005ULL+1442695040888963407ULL; h[i]=(int)((s>>33)%rows);} cudaMemcpy(kk,h.data(),nnz*4,cudaMemcpyHostToDevice);
    for (int bpsm : {4, 8, 16}) {
      int grid=sms*bpsm;
      gather_kernel<<<grid,256>>>(B,C,jj,kk,nnz,out);
      cudaEventRecord(e0); gather_kernel<<<grid,256>>>(B,C,jj,kk,nnz,out); cudaEventRecord(e1); CK(cudaEventSynchronize(e1));
      cudaEventElapsedTime(&ms,e0,e1);
      printf("gather rows=%lld (%.1f MB/table) bpsm%d: %.3f ms, %.2f Gnnz/s, gathered %.1f GB/s\n", (long long)rows, rows*256/1e6, bpsm, ms, nnz/ms/1e6, nnz*512.0/ms/1e6);
    }
    cudaFree(B); cudaFree(C);
  }
  int64_t n2 = (1LL<<30)/16; double2 *a,*b; CK(cudaMalloc(&a,n2*16)); CK(cudaMalloc(&b,n2*16));
  copy_kernel<<<sms*8,256>>>(a,b,n2);
  cudaEventRecord(e0); copy_kernel<<<sms*8,256>>>(a,b,n2); cudaEventRecord(e1); CK(cudaEventSynchronize(e1));
  cudaEventElapsedTime(&ms,e0,e1); printf("copy 1GiB: %.1f GB/s\n", 2.0*n2*16/ms/1e6);
  return 0;
}
