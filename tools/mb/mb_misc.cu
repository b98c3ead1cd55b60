// Throwaway microbenchmarks (round 1): shared-memory atomic throughput for pass-A style
// per-kernel moment tables, and FP64 pipe throughput. Not part of the product.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
#define CK(x) do{cudaError_t e=(x); if(e){printf("err %s line %d\n",cudaGetErrorString(e),__LINE__); return 1;}}while(0)
typedef unsigned long long u64;
__device__ __forceinline__ u64 mix(u64 z){z+=0x9E3779B97F4A7C15ull;z=(z^(z>>30))*0xBF58476D1CE4E5B9ull;z=(z^(z>>27))*0x94D049BB133111EBull;return z^(z>>31);}
__global__ void gen(uint32_t* kid, u64* x, size_t n, int K){
  for(size_t i=blockIdx.x*(size_t)blockDim.x+threadIdx.x;i<n;i+=(size_t)gridDim.x*blockDim.x){
    u64 h=mix(i); unsigned u=(unsigned)(h>>40); // zipf-ish: kid = K^(u/2^24) - 1 approx via sqrt trick
    float f=__powf((float)K, (float)u/16777216.0f); unsigned k=(unsigned)f-1; if(k>=K)k=K-1;
    kid[i]=k; x[i]=(mix(h)&((1ull<<40)-1))+1; }
}
__global__ void stream_read(const uint32_t* kid,const u64* x,size_t n,u64* out){
  u64 acc=0; for(size_t i=blockIdx.x*(size_t)blockDim.x+threadIdx.x;i<n;i+=(size_t)gridDim.x*blockDim.x) acc+=x[i]^kid[i];
  if(acc==42) out[0]=acc;
}
// (a) u32 shared atomics: n, and S1 in 3 x 16-bit-ish limbs (flush per chunk)
template<int MODE>
__global__ void hist(const uint32_t* kid,const u64* x,size_t n,int K,u64* g){
  extern __shared__ unsigned char sm[];
  unsigned* cnt=(unsigned*)sm; unsigned* l0=cnt+K; unsigned* l1=l0+K; unsigned* l2=l1+K; unsigned* l3=l2+K;
  u64* s64=(u64*)(sm); u64* s64b=s64+K; u64* s64c=s64b+K;
  for(int i=threadIdx.x;i<5*K;i+=blockDim.x) cnt[i]=0; __syncthreads();
  size_t per=(n+gridDim.x-1)/gridDim.x; size_t b=blockIdx.x*per, e=min(n,b+per);
  for(size_t i=b+threadIdx.x;i<e;i+=blockDim.x){ unsigned k=kid[i]; u64 v=x[i];
    if(MODE==0){ atomicAdd(&cnt[k],1u); atomicAdd(&l0[k],(unsigned)(v&0xFFFFF)); atomicAdd(&l1[k],(unsigned)((v>>20)&0xFFFFF)); atomicAdd(&l2[k],(unsigned)(v>>40)); atomicAdd(&l3[k],(unsigned)(v&0xFFF));}
    else if(MODE==1){ atomicAdd(&s64[k],v); atomicAdd(&s64b[k],v*v); atomicAdd(&s64c[k],v>>3);}  // CAS-spin u64
    else if(MODE==3){ unsigned peers=__match_any_sync(__activemask(),k); int lead=__ffs(peers)-1; unsigned lane=threadIdx.x&31;
      unsigned c=__popc(peers); if(lane==lead){atomicAdd(&cnt[k],c);} atomicAdd(&l0[k],(unsigned)(v&0xFFFFF)); }
    else if(MODE==4){ atomicAdd(&cnt[k],1u); }
    else { atomicAdd(&g[k],v); atomicAdd(&g[K+k],v*v); atomicAdd(&g[2*K+k],1ull);} // global RED
  }
  __syncthreads(); if(MODE<2) for(int i=threadIdx.x;i<K;i+=blockDim.x) atomicAdd(&g[i],(u64)cnt[i]);
}
__global__ void dfma(double* out,int iters){
  double a=threadIdx.x*1e-3, b=1.0000001, c=1e-9, a2=a+1, a3=a+2, a4=a+3;
  for(int i=0;i<iters;i++){ a=fma(a,b,c); a2=fma(a2,b,c); a3=fma(a3,b,c); a4=fma(a4,b,c);}
  if(a+a2+a3+a4==1.2345) out[0]=a;
}
int main(){
  size_t n=100000000; int K=2000; uint32_t* kid; u64* x; u64* g; double* d;
  CK(cudaMalloc(&kid,n*4)); CK(cudaMalloc(&x,n*8)); CK(cudaMalloc(&g,3*K*8)); CK(cudaMalloc(&d,8));
  gen<<<148*8,256>>>(kid,x,n,K); CK(cudaDeviceSynchronize());
  cudaEvent_t a,b; cudaEventCreate(&a); cudaEventCreate(&b); float ms;
  for(int r=0;r<3;r++){ cudaEventRecord(a); stream_read<<<148*8,512>>>(kid,x,n,g); cudaEventRecord(b); cudaEventSynchronize(b); cudaEventElapsedTime(&ms,a,b);}
  printf("stream read 12B/inv: %.3f ms  %.1f GB/s\n",ms,n*12/ms/1e6);
  int smem=6*K*8; 
  CK(cudaFuncSetAttribute(hist<0>,cudaFuncAttributeMaxDynamicSharedMemorySize,smem));
  CK(cudaFuncSetAttribute(hist<1>,cudaFuncAttributeMaxDynamicSharedMemorySize,smem));
  CK(cudaFuncSetAttribute(hist<2>,cudaFuncAttributeMaxDynamicSharedMemorySize,smem));
  CK(cudaFuncSetAttribute(hist<3>,cudaFuncAttributeMaxDynamicSharedMemorySize,smem));
  CK(cudaFuncSetAttribute(hist<4>,cudaFuncAttributeMaxDynamicSharedMemorySize,smem));
  for(int occ=1;occ<=2;occ*=2) for(int m=0;m<5;m++){ for(int r=0;r<3;r++){ cudaEventRecord(a);
      if(m==0) hist<0><<<148*occ,512,smem>>>(kid,x,n,K,g); else if(m==1) hist<1><<<148*occ,512,smem>>>(kid,x,n,K,g); else if(m==2) hist<2><<<148*occ,512,smem>>>(kid,x,n,K,g); else if(m==3) hist<3><<<148*occ,512,smem>>>(kid,x,n,K,g); else hist<4><<<148*occ,512,smem>>>(kid,x,n,K,g);
      cudaEventRecord(b); cudaEventSynchronize(b); cudaEventElapsedTime(&ms,a,b);} CK(cudaGetLastError());
    printf("hist mode %d occ %d: %.3f ms  (%.2f ns per inv per SM => atomics/clk/SM...)\n",m,occ,ms, ms*1e6/ (n/148.0)); }
  for(int r=0;r<3;r++){ cudaEventRecord(a); dfma<<<148*8,256>>>(d,100000); cudaEventRecord(b); cudaEventSynchronize(b); cudaEventElapsedTime(&ms,a,b);}
  double fl=148.0*8*256*100000*4*2; printf("DFMA: %.3f ms %.2f TFLOP/s (%.1f DFMA/clk/SM at 1.965GHz)\n",ms,fl/ms/1e9, fl/2/(ms*1e-3)/148/1.965e9);
  return 0;
}
