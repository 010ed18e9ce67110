// Throwaway microbenchmarks: atomic / gather throughput on B200 (design input only).
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
#define CK(x) do{cudaError_t e=(x); if(e!=cudaSuccess){printf("err %s line %d\n",cudaGetErrorString(e),__LINE__);return 1;}}while(0)
__device__ __forceinline__ uint32_t hsh(uint32_t x){x^=x>>16;x*=0x7feb352d;x^=x>>15;x*=0x846ca68b;x^=x>>16;return x;}
// mode 0: random over region; mode 1: clustered (each warp within window of W elems)
__global__ void k_red64(unsigned long long* a, uint32_t n_elems, uint32_t nops, int mode, uint32_t win){
  uint32_t tid=blockIdx.x*blockDim.x+threadIdx.x, nt=gridDim.x*blockDim.x;
  for(uint32_t i=tid;i<nops;i+=nt){
    uint32_t idx;
    if(mode==0) idx=hsh(i)%n_elems; else { uint32_t w=i>>5; idx=((hsh(w)%(n_elems/win))*win + (hsh(i)%win)); }
    atomicAdd(a+idx, 1ull);
  }
}
__global__ void k_red32f(float* a, uint32_t n_elems, uint32_t nops, int mode, uint32_t win){
  uint32_t tid=blockIdx.x*blockDim.x+threadIdx.x, nt=gridDim.x*blockDim.x;
  for(uint32_t i=tid;i<nops;i+=nt){
    uint32_t idx;
    if(mode==0) idx=hsh(i)%n_elems; else { uint32_t w=i>>5; idx=((hsh(w)%(n_elems/win))*win + (hsh(i)%win)); }
    atomicAdd(a+idx, 1.0f);
  }
}
__global__ void k_red32u(unsigned* a, uint32_t n_elems, uint32_t nops, int mode, uint32_t win){
  uint32_t tid=blockIdx.x*blockDim.x+threadIdx.x, nt=gridDim.x*blockDim.x;
  for(uint32_t i=tid;i<nops;i+=nt){
    uint32_t idx;
    if(mode==0) idx=hsh(i)%n_elems; else { uint32_t w=i>>5; idx=((hsh(w)%(n_elems/win))*win + (hsh(i)%win)); }
    atomicAdd(a+idx, 1u);
  }
}
template<typename T>
__global__ void k_smem_atom(T* out, uint32_t nops_per_block, uint32_t win){
  extern __shared__ __align__(16) unsigned char sm[];
  T* s=(T*)sm;
  for(uint32_t i=threadIdx.x;i<win;i+=blockDim.x) s[i]=0;
  __syncthreads();
  uint32_t base=blockIdx.x*nops_per_block;
  for(uint32_t i=threadIdx.x;i<nops_per_block;i+=blockDim.x){
    uint32_t idx=hsh(base+i)%win;
    atomicAdd(s+idx,(T)1);
  }
  __syncthreads();
  T acc=0; for(uint32_t i=threadIdx.x;i<win;i+=blockDim.x) acc+=s[i];
  if(acc==(T)12345) out[0]=acc;
}
__global__ void k_gather64(const double* a, double* out, uint32_t n_elems, uint32_t nops, int mode, uint32_t win){
  uint32_t tid=blockIdx.x*blockDim.x+threadIdx.x, nt=gridDim.x*blockDim.x;
  double acc=0;
  for(uint32_t i=tid;i<nops;i+=nt){
    uint32_t idx;
    if(mode==0) idx=hsh(i)%n_elems; else { uint32_t w=i>>5; idx=((hsh(w)%(n_elems/win))*win + (hsh(i)%win)); }
    acc+=__ldg(a+idx);
  }
  if(acc==1.2345) out[0]=acc;
}
__global__ void k_copy(const float4* a, float4* b, size_t n){
  size_t tid=blockIdx.x*(size_t)blockDim.x+threadIdx.x, nt=(size_t)gridDim.x*blockDim.x;
  for(size_t i=tid;i<n;i+=nt) b[i]=a[i];
}
int main(){
  int dev=0; cudaDeviceProp p; CK(cudaGetDeviceProperties(&p,dev));
  printf("dev %s SMs %d L2 %d MB smemPerBlockOptin %zu\n",p.name,p.multiProcessorCount,p.l2CacheSize>>20,p.sharedMemPerBlockOptin);
  cudaEvent_t e0,e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  float ms;
  size_t bigN = 1ull<<28; // 1 GiB of floats (4 B) -> 2 arrays 1 GiB each
  float4 *ca,*cb; CK(cudaMalloc(&ca,bigN*4)); CK(cudaMalloc(&cb,bigN*4));
  cudaMemset(ca,0,bigN*4);
  for(int r=0;r<3;r++){ cudaEventRecord(e0); k_copy<<<148*8,512>>>(ca,cb,bigN/4); cudaEventRecord(e1); cudaEventSynchronize(e1);}
  cudaEventElapsedTime(&ms,e0,e1); printf("copy: %.1f GB/s\n", 2.0*bigN*4/ms/1e6);
  uint32_t nops=40000000;
  unsigned long long* a64; CK(cudaMalloc(&a64, (size_t)64<<20));
  uint32_t sizes[]={1u<<20, 2u<<20, 4u<<20}; // elements of 8B: 8,16,32 MB
  for(uint32_t ne: sizes){
    for(int mode=0;mode<2;mode++){ for(uint32_t win: {32u,256u,4096u}){ if(mode==0&&win!=32u) continue;
      cudaMemset(a64,0,(size_t)ne*8);
      for(int r=0;r<3;r++){cudaEventRecord(e0); k_red64<<<148*16,256>>>(a64,ne,nops,mode,win); cudaEventRecord(e1); cudaEventSynchronize(e1);}
      cudaEventElapsedTime(&ms,e0,e1); printf("red.u64 region %u MB mode %d win %u: %.2f Gop/s (%.1f us for 4e7)\n", ne*8>>20, mode, win, nops/ms/1e6, ms*1e3);
    }}
  }
  float* af=(float*)a64; unsigned* au=(unsigned*)a64;
  for(int mode=0;mode<2;mode++){ for(uint32_t win: {32u,256u}){ if(mode==0&&win!=32u) continue;
    for(int r=0;r<3;r++){cudaEventRecord(e0); k_red32f<<<148*16,256>>>(af,2u<<20,nops,mode,win); cudaEventRecord(e1); cudaEventSynchronize(e1);}
    cudaEventElapsedTime(&ms,e0,e1); printf("red.f32 8MB mode %d win %u: %.2f Gop/s\n", mode,win, nops/ms/1e6);
    for(int r=0;r<3;r++){cudaEventRecord(e0); k_red32u<<<148*16,256>>>(au,2u<<20,nops,mode,win); cudaEventRecord(e1); cudaEventSynchronize(e1);}
    cudaEventElapsedTime(&ms,e0,e1); printf("red.u32 8MB mode %d win %u: %.2f Gop/s\n", mode,win, nops/ms/1e6);
  }}
  // smem atomics
  uint32_t nb=148*8, per=nops/nb;
  for(uint32_t win: {1024u, 4096u}){
    cudaFuncSetAttribute(k_smem_atom<unsigned long long>, cudaFuncAttributeMaxDynamicSharedMemorySize, 64*1024);
    for(int r=0;r<3;r++){cudaEventRecord(e0); k_smem_atom<unsigned long long><<<nb,256,win*8>>>(a64,per,win); cudaEventRecord(e1); cudaEventSynchronize(e1);}
    cudaEventElapsedTime(&ms,e0,e1); printf("smem atom u64 win %u: %.2f Gop/s\n", win, (double)per*nb/ms/1e6);
    for(int r=0;r<3;r++){cudaEventRecord(e0); k_smem_atom<unsigned><<<nb,256,win*4>>>((unsigned*)a64,per,win); cudaEventRecord(e1); cudaEventSynchronize(e1);}
    cudaEventElapsedTime(&ms,e0,e1); printf("smem atom u32 win %u: %.2f Gop/s\n", win, (double)per*nb/ms/1e6);
    for(int r=0;r<3;r++){cudaEventRecord(e0); k_smem_atom<float><<<nb,256,win*4>>>((float*)a64,per,win); cudaEventRecord(e1); cudaEventSynchronize(e1);}
    cudaEventElapsedTime(&ms,e0,e1); printf("smem atom f32 win %u: %.2f Gop/s\n", win, (double)per*nb/ms/1e6);
  }
  double* d64=(double*)a64; double* dout; cudaMalloc(&dout,64);
  for(uint32_t ne: sizes){ for(int mode=0;mode<2;mode++){ for(uint32_t win: {32u,256u,4096u}){ if(mode==0&&win!=32u) continue;
    for(int r=0;r<3;r++){cudaEventRecord(e0); k_gather64<<<148*16,256>>>(d64,dout,ne,nops,mode,win); cudaEventRecord(e1); cudaEventSynchronize(e1);}
    cudaEventElapsedTime(&ms,e0,e1); printf("gather f64 region %u MB mode %d win %u: %.2f Gop/s\n", ne*8>>20, mode, win, nops/ms/1e6);
  }}}
  CK(cudaGetLastError());
  return 0;
}
