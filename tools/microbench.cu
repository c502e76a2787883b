// Design-probe microbenchmarks for the construction kernels (not product code).
// Measures: HBM streaming read, smem atomicAdd / atomicCAS on spread addresses,
// global red.add to an L2-resident array, random 4 B gathers from L2.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
#define CK(x) do{cudaError_t e=(x); if(e){printf("err %s line %d\n",cudaGetErrorString(e),__LINE__); return 1;}}while(0)

__device__ __forceinline__ uint32_t hsh(uint32_t x){ x^=x>>16; x*=0x7feb352dU; x^=x>>15; x*=0x846ca68bU; x^=x>>16; return x; }

__global__ void k_stream(const int4* __restrict__ a, size_t n4, int* out){
  int4 acc = make_int4(0,0,0,0);
  for(size_t i = blockIdx.x*(size_t)blockDim.x + threadIdx.x; i < n4; i += (size_t)gridDim.x*blockDim.x){
    int4 v = __ldg(a+i); acc.x^=v.x; acc.y^=v.y; acc.z^=v.z; acc.w^=v.w; }
  if((acc.x^acc.y^acc.z^acc.w)==0x12345) out[0]=1;
}
template<int MODE>
__global__ void k_smem_atom(int iters, int* out){
  __shared__ int tab[8192];
  for(int i=threadIdx.x;i<8192;i+=blockDim.x) tab[i]=0;
  __syncthreads();
  uint32_t s = hsh(threadIdx.x + blockIdx.x*1024);
  for(int it=0; it<iters; ++it){
    s = hsh(s); uint32_t idx = s & 8191;
    if(MODE==0) atomicAdd(&tab[idx], 1);
    else if(MODE==1) atomicCAS(&tab[idx], 0, 1);
    else if(MODE==2) { tab[idx] += 1; }
  }
  __syncthreads();
  if(threadIdx.x==0) out[blockIdx.x] = tab[5];
}
__global__ void k_gred(int* arr, uint32_t mask, int iters){
  uint32_t s = hsh(threadIdx.x + blockIdx.x*1024);
  for(int it=0; it<iters; ++it){ s = hsh(s); atomicAdd(&arr[s & mask], 1); }
}
__global__ void k_gather(const int* __restrict__ arr, uint32_t mask, int iters, int* out){
  uint32_t s = hsh(threadIdx.x + blockIdx.x*1024); int acc=0;
  for(int it=0; it<iters; it+=4){
    uint32_t s1=hsh(s), s2=hsh(s1), s3=hsh(s2), s4=hsh(s3); s=s4;
    acc += __ldg(arr+(s1&mask)) + __ldg(arr+(s2&mask)) + __ldg(arr+(s3&mask)) + __ldg(arr+(s4&mask)); }
  if(acc==0x1234567) out[0]=acc;
}
int main(){
  cudaDeviceProp p; CK(cudaGetDeviceProperties(&p,0));
  printf("device %s SMs %d L2 %d MB smem/blk optin %zu clock %d\n", p.name, p.multiProcessorCount, p.l2CacheSize>>20, p.sharedMemPerBlockOptin, p.clockRate);
  int nsm = p.multiProcessorCount;
  cudaEvent_t e0,e1; cudaEventCreate(&e0); cudaEventCreate(&e1); float ms;
  size_t bytes = (size_t)8<<30; int4* a; CK(cudaMalloc(&a, bytes)); CK(cudaMemset(a, 1, bytes));
  int* out; CK(cudaMalloc(&out, 1<<20));
  for(int rep=0;rep<3;rep++){
    cudaEventRecord(e0); k_stream<<<nsm*8,512>>>(a, bytes/16, out); cudaEventRecord(e1); CK(cudaEventSynchronize(e1));
    cudaEventElapsedTime(&ms,e0,e1); printf("stream read 8GB: %.3f ms -> %.1f GB/s\n", ms, bytes/ms/1e6);
  }
  const char* names[3]={"smem atomicAdd","smem atomicCAS","smem plain rmw"};
  for(int mode=0;mode<3;mode++){
    int iters=4096; int blocks=nsm*4, thr=512;
    for(int rep=0;rep<2;rep++){
      cudaEventRecord(e0);
      if(mode==0) k_smem_atom<0><<<blocks,thr>>>(iters,out);
      if(mode==1) k_smem_atom<1><<<blocks,thr>>>(iters,out);
      if(mode==2) k_smem_atom<2><<<blocks,thr>>>(iters,out);
      cudaEventRecord(e1); CK(cudaEventSynchronize(e1)); cudaEventElapsedTime(&ms,e0,e1);
      double ops=(double)blocks*thr*iters; printf("%s: %.3f ms, %.2f Gop/s, %.3f op/clk/SM\n", names[mode], ms, ops/ms/1e6, ops/(ms*1e-3)/(p.clockRate*1e3)/nsm);
    }
  }
  int* arr; CK(cudaMalloc(&arr, (size_t)64<<20)); CK(cudaMemset(arr,0,(size_t)64<<20));
  for(uint32_t mask : {(1u<<12)-1,(1u<<20)-1,(1u<<24)-1}){
    int iters=1024, blocks=nsm*8, thr=512;
    for(int rep=0;rep<2;rep++){
      cudaEventRecord(e0); k_gred<<<blocks,thr>>>(arr,mask,iters); cudaEventRecord(e1); CK(cudaEventSynchronize(e1)); cudaEventElapsedTime(&ms,e0,e1);
      double ops=(double)blocks*thr*iters; printf("global atomicAdd range %u: %.3f ms %.2f Gop/s\n", mask+1, ms, ops/ms/1e6);
    }
    for(int rep=0;rep<2;rep++){
      cudaEventRecord(e0); k_gather<<<blocks,thr>>>(arr,mask,iters,out); cudaEventRecord(e1); CK(cudaEventSynchronize(e1)); cudaEventElapsedTime(&ms,e0,e1);
      double ops=(double)blocks*thr*iters; printf("random gather range %u: %.3f ms %.2f Gop/s\n", mask+1, ms, ops/ms/1e6);
    }
  }
  return 0;
}
