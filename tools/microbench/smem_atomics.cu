// Microbenchmarks that decide the accumulator design:
// throughput of the shared-memory and L2 primitives a Gustavson accumulator can be built from.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o mb smem_atomics.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
#define CK(x) do{cudaError_t e=(x); if(e!=cudaSuccess){printf("CUDA %s at %d\n",cudaGetErrorString(e),__LINE__); return 1;}}while(0)

constexpr int ITERS = 4096;
__device__ __forceinline__ uint32_t lcg(uint32_t& x){ x = x*1664525u + 1013904223u; return x; }

// 1: fp64 atomicAdd on smem (compiles to a CAS spin loop), random addresses over NS doubles
template<int NS> __global__ void k_cas_f64(double* out){
  extern __shared__ double s[];
  for(int i=threadIdx.x;i<NS;i+=blockDim.x) s[i]=0; __syncthreads();
  uint32_t x = blockIdx.x*blockDim.x+threadIdx.x;
  for(int it=0;it<ITERS;++it){ atomicAdd(&s[(lcg(x)>>8)&(NS-1)], 1.0); }
  __syncthreads(); if(threadIdx.x==0) out[blockIdx.x]=s[0];
}
// 2: plain LDS/DADD/STS on warp-private region; lanes have distinct addresses (lane + 32*r)
template<int NS> __global__ void k_rmw_f64(double* out){
  extern __shared__ double s[];
  for(int i=threadIdx.x;i<NS*(blockDim.x/32);i+=blockDim.x) s[i]=0; __syncthreads();
  double* w = s + (threadIdx.x/32)*NS; int lane=threadIdx.x&31;
  uint32_t x = blockIdx.x*blockDim.x+threadIdx.x;
  for(int it=0;it<ITERS;++it){ int c = (((lcg(x)>>8)&(NS/32-1))*32) + lane; w[c] += 1.0; __syncwarp(); }
  __syncthreads(); if(threadIdx.x==0) out[blockIdx.x]=s[0];
}
// 2b: same but random column (bank conflicts as in a real gather): distinct-by-construction via c = r ^ lane*?; use random per lane within its own 1/32 slice
template<int NS> __global__ void k_rmw_f64_rand(double* out){
  extern __shared__ double s[];
  for(int i=threadIdx.x;i<NS*(blockDim.x/32);i+=blockDim.x) s[i]=0; __syncthreads();
  double* w = s + (threadIdx.x/32)*NS; int lane=threadIdx.x&31;
  uint32_t x = blockIdx.x*blockDim.x+threadIdx.x;
  for(int it=0;it<ITERS;++it){ int c = lane*(NS/32) + ((lcg(x)>>8)&(NS/32-1)); w[c] += 1.0; __syncwarp(); }
  __syncthreads(); if(threadIdx.x==0) out[blockIdx.x]=s[0];
}
// 3: atomicOr 32-bit random
template<int NS> __global__ void k_or32(double* out){
  extern __shared__ uint32_t su[];
  for(int i=threadIdx.x;i<NS;i+=blockDim.x) su[i]=0; __syncthreads();
  uint32_t x = blockIdx.x*blockDim.x+threadIdx.x;
  for(int it=0;it<ITERS;++it){ uint32_t r=lcg(x); atomicOr(&su[(r>>8)&(NS-1)], 1u<<(r&31)); }
  __syncthreads(); if(threadIdx.x==0) out[blockIdx.x]=su[0];
}
// 4: atomicCAS 32-bit random (hash insert pattern; result used)
template<int NS> __global__ void k_cas32(double* out){
  extern __shared__ uint32_t su[];
  for(int i=threadIdx.x;i<NS;i+=blockDim.x) su[i]=0xffffffffu; __syncthreads();
  uint32_t x = blockIdx.x*blockDim.x+threadIdx.x; uint32_t acc=0;
  for(int it=0;it<ITERS;++it){ uint32_t r=lcg(x); uint32_t k=(r>>8)&(NS-1); acc += atomicCAS(&su[k], 0xffffffffu, k); }
  __syncthreads(); if(threadIdx.x==0) out[blockIdx.x]=acc;
}
// 5: atomicAdd int32 random
template<int NS> __global__ void k_add32(double* out){
  extern __shared__ uint32_t su[];
  for(int i=threadIdx.x;i<NS;i+=blockDim.x) su[i]=0; __syncthreads();
  uint32_t x = blockIdx.x*blockDim.x+threadIdx.x;
  for(int it=0;it<ITERS;++it){ atomicAdd(&su[(lcg(x)>>8)&(NS-1)], 1u); }
  __syncthreads(); if(threadIdx.x==0) out[blockIdx.x]=su[0];
}
// 6: byte store random (idempotent bytemap)
template<int NS> __global__ void k_st8(double* out){
  extern __shared__ uint8_t sb[];
  for(int i=threadIdx.x;i<NS;i+=blockDim.x) sb[i]=0; __syncthreads();
  uint32_t x = blockIdx.x*blockDim.x+threadIdx.x;
  for(int it=0;it<ITERS;++it){ volatile uint8_t* p = sb + ((lcg(x)>>8)&(NS-1)); *p = 1; }
  __syncthreads(); if(threadIdx.x==0) out[blockIdx.x]=sb[0];
}
// 7: global RED.ADD.F64 random into region of R doubles
__global__ void k_red_f64(double* g, uint32_t mask){
  uint32_t x = blockIdx.x*blockDim.x+threadIdx.x;
  for(int it=0;it<ITERS/8;++it){ atomicAdd(&g[(lcg(x)>>4)&mask], 1.0); }
}
// 8: match_any throughput
__global__ void k_match(double* out){
  uint32_t x = blockIdx.x*blockDim.x+threadIdx.x; uint32_t acc=0;
  for(int it=0;it<ITERS;++it){ acc += __match_any_sync(0xffffffffu, (lcg(x)>>20)); }
  if(acc==7) out[0]=acc;
}
// 9: random 12-byte gather (col int32 + val fp64) from arrays of N entries
__global__ void k_gather(const int* __restrict__ col, const double* __restrict__ val, uint32_t mask, double* out){
  uint32_t x = blockIdx.x*blockDim.x+threadIdx.x; double acc=0;
  for(int it=0;it<ITERS/16;++it){ uint32_t q=(lcg(x)>>2)&mask; acc += val[q]*col[q]; }
  if(acc==-1) out[0]=acc;
}
// 10: coalesced segment gather: each warp reads 32 consecutive entries at a random start (B-row segment pattern)
__global__ void k_seg(const int* __restrict__ col, const double* __restrict__ val, uint32_t mask, double* out){
  uint32_t x = blockIdx.x*blockDim.x/32+threadIdx.x/32; int lane=threadIdx.x&31; double acc=0;
  for(int it=0;it<ITERS/16;++it){ uint32_t q=((lcg(x)>>2)&mask&~31u)+lane; acc += val[q]*col[q]; }
  if(acc==-1) out[0]=acc;
}

template<class F> float timeit(F f){
  cudaEvent_t a,b; cudaEventCreate(&a); cudaEventCreate(&b);
  f(); cudaDeviceSynchronize();
  cudaEventRecord(a); for(int r=0;r<5;++r) f(); cudaEventRecord(b); cudaEventSynchronize(b);
  float ms; cudaEventElapsedTime(&ms,a,b); return ms/5;
}
int main(){
  cudaDeviceProp p; CK(cudaGetDeviceProperties(&p,0));
  int clk=0; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  printf("{\"name\":\"%s\",\"sms\":%d,\"smem_per_sm\":%zu,\"smem_optin\":%zu,\"l2\":%d,\"hbm\":%zu,\"clock_khz\":%d,\"cc\":\"%d.%d\"}\n",
    p.name,p.multiProcessorCount,p.sharedMemPerMultiprocessor,p.sharedMemPerBlockOptin,p.l2CacheSize,p.totalGlobalMem,clk,p.major,p.minor);
  int SM=p.multiProcessorCount; double* out; CK(cudaMalloc(&out, 1<<20));
  const int T=512; int G=SM*2;
  auto rep=[&](const char* n, float ms, double ops){ printf("%-28s %8.3f ms  %8.2f Gop/s  %6.2f op/SM/ns\n", n, ms, ops/ms/1e6, ops/ms/1e6/SM); };
  double ops = double(G)*T*ITERS;
  #define RUN(name, K, smem) { auto f=[&]{ K<<<G,T,smem>>>(out); }; CK(cudaFuncSetAttribute(K, cudaFuncAttributeMaxDynamicSharedMemorySize, 100000)); float ms=timeit(f); CK(cudaGetLastError()); rep(name, ms, ops); }
  RUN("smem_cas_f64_16K", (k_cas_f64<8192>), 8192*8);
  RUN("smem_rmw_f64_lanestride", (k_rmw_f64<512>), 512*8*16);
  RUN("smem_rmw_f64_random", (k_rmw_f64_rand<512>), 512*8*16);
  RUN("smem_or32_16K", (k_or32<16384>), 16384*4);
  RUN("smem_cas32_16K", (k_cas32<16384>), 16384*4);
  RUN("smem_add32_16K", (k_add32<16384>), 16384*4);
  RUN("smem_st8_64K", (k_st8<65536>), 65536);
  { auto f=[&]{ k_match<<<G,T>>>(out); }; float ms=timeit(f); rep("match_any", ms, ops); }
  double* g; CK(cudaMalloc(&g, size_t(1)<<30)); cudaMemset(g,0,size_t(1)<<30);
  for(uint32_t lg : {20u, 23u, 26u}) { uint32_t mask=(1u<<lg)-1; auto f=[&]{ k_red_f64<<<G*4,T>>>(g,mask); }; float ms=timeit(f);
    char nm[64]; snprintf(nm,64,"gmem_red_f64_%uMB",(8u<<lg)>>20); rep(nm, ms, double(G)*4*T*(ITERS/8)); }
  int* col; double* val; CK(cudaMalloc(&col, size_t(4)<<26)); CK(cudaMalloc(&val, size_t(8)<<26)); cudaMemset(col,0,size_t(4)<<26); cudaMemset(val,0,size_t(8)<<26);
  for(uint32_t lg : {20u, 22u, 24u, 26u}) { uint32_t mask=(1u<<lg)-1; auto f=[&]{ k_gather<<<G*4,T>>>(col,val,mask,out); }; float ms=timeit(f);
    char nm[64]; snprintf(nm,64,"gather12B_%uMB",(12u<<lg)>>20); rep(nm, ms, double(G)*4*T*(ITERS/16)); }
  for(uint32_t lg : {20u, 22u, 24u, 26u}) { uint32_t mask=(1u<<lg)-1; auto f=[&]{ k_seg<<<G*4,T>>>(col,val,mask,out); }; float ms=timeit(f);
    char nm[64]; snprintf(nm,64,"seg32_12B_%uMB",(12u<<lg)>>20); rep(nm, ms, double(G)*4*T*(ITERS/16)); }
  return 0;
}
