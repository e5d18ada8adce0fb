// Microbenchmark (design probe, not product): shared-memory atomic throughput
// inside a shard-like stage-2 loop vs. a plain HBM stream, on B200.
#include <cstdio>
#include <cstdint>
#include <vector>
#include <random>
#include <cuda_runtime.h>
#define CK(x) do{cudaError_t e=(x); if(e!=cudaSuccess){printf("CUDA %s @%d\n",cudaGetErrorString(e),__LINE__); return 1;}}while(0)

constexpr int NV = 3392;  // vertices per shard (C2 |N|)

__global__ void stream_read(const uint4* __restrict__ a, size_t n, uint32_t* out){
  uint32_t acc=0; size_t i=blockIdx.x*(size_t)blockDim.x+threadIdx.x, st=(size_t)gridDim.x*blockDim.x;
  for(;i<n;i+=st){ uint4 v=a[i]; acc^=v.x^v.y^v.z^v.w; }
  if(acc==0x12345678) out[0]=acc;
}
// mode 0: atomicMin no-return; 1: LDS filter then atomicMin; 2: f32 atomicAdd (CAS);
// 3: u32 atomicAdd with return + carry (fixed point 64); 4: plain LDS/STS (non-atomic, wrong, floor)
template<int MODE>
__global__ void __launch_bounds__(512) stage2(const uint32_t* __restrict__ sv, const uint16_t* __restrict__ dst,
    const uint32_t* __restrict__ off, uint32_t* out){
  __shared__ uint32_t lo[NV+1]; __shared__ uint32_t hi[NV+1];
  for(int i=threadIdx.x;i<=NV;i+=blockDim.x){ lo[i]=MODE==0||MODE==1?~0u:0; hi[i]=0; }
  __syncthreads();
  uint32_t b=off[blockIdx.x], e=off[blockIdx.x+1];
  // 8 entries per thread per step: 2x uint4 of sv, 1x uint4 of dst (shards padded to 8)
  for(uint32_t base=b+threadIdx.x*8; base<e; base+=blockDim.x*8){
    uint4 s0=*(const uint4*)(sv+base), s1=*(const uint4*)(sv+base+4);
    uint4 dd=*(const uint4*)(dst+base);
    uint32_t v[8]={s0.x,s0.y,s0.z,s0.w,s1.x,s1.y,s1.z,s1.w};
    uint32_t d[8]={dd.x&0xffff,dd.x>>16,dd.y&0xffff,dd.y>>16,dd.z&0xffff,dd.z>>16,dd.w&0xffff,dd.w>>16};
    #pragma unroll
    for(int k=0;k<8;k++){
      if(MODE==0) atomicMin(&lo[d[k]], v[k]);
      else if(MODE==1){ if(v[k]<lo[d[k]]) atomicMin(&lo[d[k]], v[k]); }
      else if(MODE==2) atomicAdd((float*)&lo[d[k]], __uint_as_float(v[k]&0x3fffffff));
      else if(MODE==3){ uint32_t add=v[k]; uint32_t old=atomicAdd(&lo[d[k]], add); if(old+add<old) atomicAdd(&hi[d[k]],1u); }
      else { lo[d[k]]+=v[k]; }
    }
  }
  __syncthreads();
  uint32_t acc=0; for(int i=threadIdx.x;i<NV;i+=blockDim.x) acc^=lo[i]^hi[i];
  if(acc==0x12345678) out[blockIdx.x]=acc;
}

int main(){
  const int S=1430; const size_t per=48256; const size_t E=(size_t)S*per; // ~69M
  std::vector<uint32_t> off(S+1); for(int s=0;s<=S;s++) off[s]=s*per;
  std::vector<uint16_t> d(E); std::vector<uint32_t> v(E);
  std::mt19937_64 rng(1);
  for(int dist=0; dist<2; dist++){
    // dist 0: uniform dests; dist 1: skewed (20% of entries to dest 0 (a hub), rest zipf-ish)
    for(size_t i=0;i<E;i++){ uint64_t r=rng(); v[i]=(uint32_t)(r>>40); 
      if(dist==0) d[i]=(uint16_t)((r&0xffffffff)%NV);
      else { double u=((r&0xffffff)+0.5)/16777216.0; d[i]=(uint16_t)(std::min<double>(NV-1, std::pow(u,3.0)*NV)); } }
    uint32_t *dsv,*doff,*dout; uint16_t* dd; uint4* big;
    CK(cudaMalloc(&dsv,E*4)); CK(cudaMalloc(&dd,E*2)); CK(cudaMalloc(&doff,(S+1)*4)); CK(cudaMalloc(&dout,S*4));
    CK(cudaMemcpy(dsv,v.data(),E*4,cudaMemcpyHostToDevice)); CK(cudaMemcpy(dd,d.data(),E*2,cudaMemcpyHostToDevice));
    CK(cudaMemcpy(doff,off.data(),(S+1)*4,cudaMemcpyHostToDevice));
    size_t nb=(size_t)2<<30; CK(cudaMalloc(&big,nb));
    cudaEvent_t a,b; cudaEventCreate(&a); cudaEventCreate(&b); float ms;
    if(dist==0){ for(int r=0;r<3;r++){ cudaEventRecord(a); stream_read<<<148*8,512>>>(big,nb/16,dout); cudaEventRecord(b); cudaEventSynchronize(b);} cudaEventElapsedTime(&ms,a,b);
      printf("stream_read 2GiB: %.3f ms = %.1f GB/s\n",ms,nb/ms/1e6); }
    auto run=[&](auto kern,const char* name,int threads){ for(int r=0;r<4;r++){ stream_read<<<148*8,512>>>(big,nb/16/8,dout); cudaEventRecord(a); kern<<<S,threads>>>(dsv,dd,doff,dout); cudaEventRecord(b); cudaEventSynchronize(b);} cudaEventElapsedTime(&ms,a,b);
      printf("dist=%d %-28s thr=%d: %.3f ms  %.2f Gedge/s  eqBW(6B/e)=%.0f GB/s\n",dist,name,threads,ms,E/ms/1e6,E*6.0/ms/1e6); };
    for(int thr: {256,512}){
      run(stage2<0>,"atomicMin",thr); run(stage2<1>,"LDS-filter atomicMin",thr); run(stage2<2>,"f32 atomicAdd(CAS)",thr);
      run(stage2<3>,"u32 add+carry (fixed64)",thr); run(stage2<4>,"plain LDS/STS (floor)",thr);
    }
    CK(cudaGetLastError());
    cudaFree(dsv); cudaFree(dd); cudaFree(doff); cudaFree(dout); cudaFree(big);
  }
  return 0;
}
