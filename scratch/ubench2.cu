// Throwaway microbenchmarks, round 2: vector atomics, struct-of-3 atomics, ILP gathers.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
__device__ __forceinline__ uint32_t hsh(uint32_t x){x^=x>>16;x*=0x7feb352d;x^=x>>15;x*=0x846ca68b;x^=x>>16;return x;}
__device__ __forceinline__ uint32_t pick(uint32_t i,int mode,uint32_t n,uint32_t win){
  if(mode==0) return hsh(i)%n; uint32_t w=i>>5; return (hsh(w)%(n/win))*win + (hsh(i)%win);}
__global__ void k_v4f(float4* a, uint32_t n, uint32_t nops, int mode, uint32_t win){
  uint32_t tid=blockIdx.x*blockDim.x+threadIdx.x, nt=gridDim.x*blockDim.x;
  for(uint32_t i=tid;i<nops;i+=nt){ uint32_t idx=pick(i,mode,n,win);
    float* p=(float*)(a+idx);
    asm volatile("red.global.add.v4.f32 [%0], {%1,%2,%3,%4};"::"l"(p),"f"(1.f),"f"(-1.f),"f"(0.5f),"f"(0.f):"memory");
  }}
__global__ void k_s3u64(unsigned long long* a, uint32_t n, uint32_t nops, int mode, uint32_t win){
  uint32_t tid=blockIdx.x*blockDim.x+threadIdx.x, nt=gridDim.x*blockDim.x;
  for(uint32_t i=tid;i<nops;i+=nt){ uint32_t idx=pick(i,mode,n,win);
    unsigned long long* p=a+4*(size_t)idx; atomicAdd(p,1ull); atomicAdd(p+1,2ull); atomicAdd(p+2,3ull);
  }}
__global__ void k_s1u64(unsigned long long* a, uint32_t n, uint32_t nops, int mode, uint32_t win){
  uint32_t tid=blockIdx.x*blockDim.x+threadIdx.x, nt=gridDim.x*blockDim.x;
  for(uint32_t i=tid;i<nops;i+=nt){ uint32_t idx=pick(i,mode,n,win);
    unsigned long long* p=a+4*(size_t)idx; atomicAdd(p,1ull);
  }}
__global__ void k_gather_ilp(const double* a, double* out, uint32_t n, uint32_t nops, int mode, uint32_t win){
  uint32_t tid=blockIdx.x*blockDim.x+threadIdx.x, nt=gridDim.x*blockDim.x;
  double acc=0;
  uint32_t i=tid;
  for(;i+7*nt<nops;i+=8*nt){
    double v[8];
    #pragma unroll
    for(int j=0;j<8;j++) v[j]=__ldg(a+pick(i+j*nt,mode,n,win));
    #pragma unroll
    for(int j=0;j<8;j++) acc+=v[j];
  }
  if(acc==1.2345) out[0]=acc;
}
__global__ void k_gather_v4(const double4* a, double* out, uint32_t n, uint32_t nops, int mode, uint32_t win){
  uint32_t tid=blockIdx.x*blockDim.x+threadIdx.x, nt=gridDim.x*blockDim.x;
  double acc=0; uint32_t i=tid;
  for(;i+7*nt<nops;i+=8*nt){
    double4 v[8];
    #pragma unroll
    for(int j=0;j<8;j++) v[j]=a[pick(i+j*nt,mode,n,win)];
    #pragma unroll
    for(int j=0;j<8;j++) acc+=v[j].x+v[j].y+v[j].z;
  }
  if(acc==1.2345) out[0]=acc;
}
__global__ void k_smem_gather(double* out, uint32_t nops_per_block, uint32_t win){
  extern __shared__ double s[];
  for(uint32_t i=threadIdx.x;i<win;i+=blockDim.x) s[i]=i;
  __syncthreads();
  double acc=0; uint32_t base=blockIdx.x*nops_per_block;
  for(uint32_t i=threadIdx.x;i<nops_per_block;i+=blockDim.x) acc+=s[hsh(base+i)%win];
  if(acc==1.2345) out[0]=acc;
}
int main(){
  cudaEvent_t e0,e1; cudaEventCreate(&e0); cudaEventCreate(&e1); float ms;
  void* buf; cudaMalloc(&buf,(size_t)256<<20); cudaMemset(buf,0,(size_t)256<<20);
  uint32_t nops=20000000; uint32_t nv=1u<<20; // 1M vertices
  for(int mode=0;mode<2;mode++) for(uint32_t win: {32u,256u,4096u}){ if(mode==0&&win!=32u) continue;
    for(int r=0;r<3;r++){cudaEventRecord(e0); k_v4f<<<148*16,256>>>((float4*)buf,nv,nops,mode,win); cudaEventRecord(e1); cudaEventSynchronize(e1);}
    cudaEventElapsedTime(&ms,e0,e1); printf("red.v4.f32 1M vtx mode %d win %u: %.1f Gop/s\n",mode,win,nops/ms/1e6);
    for(int r=0;r<3;r++){cudaEventRecord(e0); k_s3u64<<<148*16,256>>>((unsigned long long*)buf,nv,nops,mode,win); cudaEventRecord(e1); cudaEventSynchronize(e1);}
    cudaEventElapsedTime(&ms,e0,e1); printf("3x red.u64 same sector mode %d win %u: %.1f Gvtx/s\n",mode,win,nops/ms/1e6);
    for(int r=0;r<3;r++){cudaEventRecord(e0); k_s1u64<<<148*16,256>>>((unsigned long long*)buf,nv,nops,mode,win); cudaEventRecord(e1); cudaEventSynchronize(e1);}
    cudaEventElapsedTime(&ms,e0,e1); printf("1x red.u64 stride32B mode %d win %u: %.1f Gop/s\n",mode,win,nops/ms/1e6);
  }
  double* dout; cudaMalloc(&dout,64);
  for(uint32_t ne: {1u<<20, 2u<<20}) for(int mode=0;mode<2;mode++) for(uint32_t win: {32u,256u,4096u}){ if(mode==0&&win!=32u) continue;
    for(int r=0;r<3;r++){cudaEventRecord(e0); k_gather_ilp<<<148*8,256>>>((double*)buf,dout,ne,nops*2,mode,win); cudaEventRecord(e1); cudaEventSynchronize(e1);}
    cudaEventElapsedTime(&ms,e0,e1); printf("gather f64 ILP8 %u MB mode %d win %u: %.1f Gop/s\n",ne*8>>20,mode,win,2.0*nops/ms/1e6);
  }
  for(int mode=0;mode<2;mode++) for(uint32_t win: {32u,256u}){ if(mode==0&&win!=32u) continue;
    for(int r=0;r<3;r++){cudaEventRecord(e0); k_gather_v4<<<148*8,256>>>((double4*)buf,dout,nv,nops,mode,win); cudaEventRecord(e1); cudaEventSynchronize(e1);}
    cudaEventElapsedTime(&ms,e0,e1); printf("gather double4 (32B) ILP8 1M vtx mode %d win %u: %.1f Gop/s\n",mode,win,nops/ms/1e6);
  }
  for(uint32_t win: {1024u,4096u}){
    uint32_t nb=148*8, per=(nops*2)/nb;
    for(int r=0;r<3;r++){cudaEventRecord(e0); k_smem_gather<<<nb,256,win*8>>>(dout,per,win); cudaEventRecord(e1); cudaEventSynchronize(e1);}
    cudaEventElapsedTime(&ms,e0,e1); printf("smem gather f64 win %u: %.1f Gop/s\n",win,(double)per*nb/ms/1e6);
  }
  cudaError_t e=cudaGetLastError(); printf("err: %s\n",cudaGetErrorString(e));
}
