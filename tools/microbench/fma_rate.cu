// Microbenchmark: FP32 FMA issue rate on sm_100a for the NCC numerator's inner-loop shapes.
// (a) scalar FFMA outer-product: RV independent accumulators, broadcast template scalar,
// (b) FFMA2 with a scalar (.F32) broadcast operand and RV/2 paired accumulators,
// (c) same as (a)/(b) but with operands streamed from shared memory (LDS.128 per 4 j-steps).
#include <cstdio>
#include <cuda_runtime.h>
#include <cstdint>

#define RV 12
typedef unsigned long long u64;
__device__ __forceinline__ u64 pk(float a, float b){ u64 r; asm("mov.b64 %0, {%1,%2};" : "=l"(r) : "f"(a), "f"(b)); return r; }
__device__ __forceinline__ void ffma2(u64& d, float a, u64 b){ asm volatile("fma.rn.f32x2 %0, %1, %2, %0;" : "+l"(d) : "l"(pk(a,a)), "l"(b)); }

__global__ void __launch_bounds__(256) k_ffma(float* out, const float* in, int iters){
  float acc[RV]; float x[RV];
  #pragma unroll
  for(int c=0;c<RV;c++){ acc[c]=0.f; x[c]=in[threadIdx.x+c]; }
  float t0=in[0], t1=in[1], t2=in[2], t3=in[3];
  for(int i=0;i<iters;i++){
    #pragma unroll
    for(int c=0;c<RV;c++){ acc[c]=fmaf(t0,x[c],acc[c]); }
    #pragma unroll
    for(int c=0;c<RV;c++){ acc[c]=fmaf(t1,x[(c+1)%RV],acc[c]); }
    #pragma unroll
    for(int c=0;c<RV;c++){ acc[c]=fmaf(t2,x[(c+2)%RV],acc[c]); }
    #pragma unroll
    for(int c=0;c<RV;c++){ acc[c]=fmaf(t3,x[(c+3)%RV],acc[c]); }
  }
  float s=0; 
  #pragma unroll
  for(int c=0;c<RV;c++) s+=acc[c];
  out[blockIdx.x*blockDim.x+threadIdx.x]=s;
}

__global__ void __launch_bounds__(256) k_ffma2(float* out, const float* in, int iters){
  u64 acc[RV/2]; u64 x[RV/2];
  #pragma unroll
  for(int c=0;c<RV/2;c++){ acc[c]=pk(0.f,0.f); x[c]=pk(in[threadIdx.x+c], in[threadIdx.x+c+RV/2]); }
  float t0=in[0], t1=in[1], t2=in[2], t3=in[3];
  for(int i=0;i<iters;i++){
    #pragma unroll
    for(int c=0;c<RV/2;c++) ffma2(acc[c], t0, x[c]);
    #pragma unroll
    for(int c=0;c<RV/2;c++) ffma2(acc[c], t1, x[(c+1)%(RV/2)]);
    #pragma unroll
    for(int c=0;c<RV/2;c++) ffma2(acc[c], t2, x[(c+2)%(RV/2)]);
    #pragma unroll
    for(int c=0;c<RV/2;c++) ffma2(acc[c], t3, x[(c+3)%(RV/2)]);
  }
  float s=0;
  #pragma unroll
  for(int c=0;c<RV/2;c++){ float2 f=*reinterpret_cast<float2*>(&acc[c]); s+=f.x+f.y; }
  out[blockIdx.x*blockDim.x+threadIdx.x]=s;
}

// smem-fed sliding window, scalar FFMA: per 4 j-steps one LDS.128 image + one LDS.128 template (broadcast)
__global__ void __launch_bounds__(256) k_smem_ffma(float* out, const float* in, int iters){
  __shared__ __align__(16) float img[8][8*RV+64+4];
  __shared__ __align__(16) float tpl[64];
  int lane=threadIdx.x&31, w=threadIdx.x>>5;
  for(int k=threadIdx.x;k<8*(8*RV+68);k+=256) (&img[0][0])[k]=in[k&1023];
  if(threadIdx.x<64) tpl[threadIdx.x]=in[threadIdx.x+5];
  __syncthreads();
  const float* row=&img[(lane>>3)+ (w&4)][(lane&7)*RV];
  float acc[RV];
  #pragma unroll
  for(int c=0;c<RV;c++) acc[c]=0.f;
  for(int i=0;i<iters;i++){
    float x[RV];
    #pragma unroll
    for(int c=0;c<RV;c+=4){ float4 v=*reinterpret_cast<const float4*>(row+c); x[c]=v.x;x[c+1]=v.y;x[c+2]=v.z;x[c+3]=v.w; }
    #pragma unroll
    for(int j=0;j<64;j+=4){
      float4 nx=*reinterpret_cast<const float4*>(row+RV+j);
      float4 t=*reinterpret_cast<const float4*>(tpl+j);
      float tt[4]={t.x,t.y,t.z,t.w}; float nn[4]={nx.x,nx.y,nx.z,nx.w};
      #pragma unroll
      for(int s=0;s<4;s++){
        #pragma unroll
        for(int c=0;c<RV;c++) acc[c]=fmaf(tt[s],x[c],acc[c]);
        #pragma unroll
        for(int c=0;c<RV-1;c++) x[c]=x[c+1];
        x[RV-1]=nn[s];
      }
    }
  }
  float s=0;
  #pragma unroll
  for(int c=0;c<RV;c++) s+=acc[c];
  out[blockIdx.x*blockDim.x+threadIdx.x]=s;
}

// smem-fed sliding window, FFMA2 with column pairs (c, c+RV/2) stored interleaved in smem
__global__ void __launch_bounds__(256) k_smem_ffma2(float* out, const float* in, int iters){
  __shared__ __align__(16) float2 img[8][8*RV+64+4];
  __shared__ __align__(16) float tpl[64];
  int lane=threadIdx.x&31, w=threadIdx.x>>5;
  for(int k=threadIdx.x;k<8*(8*RV+68);k+=256) (&img[0][0])[k]=make_float2(in[k&1023], in[(k+7)&1023]);
  if(threadIdx.x<64) tpl[threadIdx.x]=in[threadIdx.x+5];
  __syncthreads();
  const float2* row=&img[(lane>>3)+(w&4)][(lane&7)*(RV/2)];
  u64 acc[RV/2];
  #pragma unroll
  for(int c=0;c<RV/2;c++) acc[c]=0ull;
  for(int i=0;i<iters;i++){
    u64 x[RV/2];
    #pragma unroll
    for(int c=0;c<RV/2;c++) x[c]=*reinterpret_cast<const u64*>(row+c);
    #pragma unroll
    for(int j=0;j<64;j+=4){
      ulonglong2 n01=*reinterpret_cast<const ulonglong2*>(row+RV/2+j);
      ulonglong2 n23=*reinterpret_cast<const ulonglong2*>(row+RV/2+j+2);
      float4 t=*reinterpret_cast<const float4*>(tpl+j);
      float tt[4]={t.x,t.y,t.z,t.w}; u64 nn[4]={n01.x,n01.y,n23.x,n23.y};
      #pragma unroll
      for(int s=0;s<4;s++){
        #pragma unroll
        for(int c=0;c<RV/2;c++) ffma2(acc[c],tt[s],x[c]);
        #pragma unroll
        for(int c=0;c<RV/2-1;c++) x[c]=x[c+1];
        x[RV/2-1]=nn[s];
      }
    }
  }
  float s=0;
  #pragma unroll
  for(int c=0;c<RV/2;c++){ float2 f=*reinterpret_cast<float2*>(&acc[c]); s+=f.x+f.y; }
  out[blockIdx.x*blockDim.x+threadIdx.x]=s;
}

template<typename K>
void run(const char* name, K kern, double fma_per_thread_iter, int iters, int blocks, float* out, const float* in){
  cudaEvent_t a,b; cudaEventCreate(&a); cudaEventCreate(&b);
  kern<<<blocks,256>>>(out,in,iters); cudaDeviceSynchronize();
  cudaEventRecord(a);
  for(int r=0;r<5;r++) kern<<<blocks,256>>>(out,in,iters);
  cudaEventRecord(b); cudaEventSynchronize(b);
  float ms; cudaEventElapsedTime(&ms,a,b); ms/=5;
  double flop=2.0*fma_per_thread_iter*iters*blocks*256.0;
  int clk; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  printf("%-14s %8.3f ms  %7.2f TFLOP/s  (nominal peak @%d MHz: %.2f)\n", name, ms, flop/ms/1e9, clk/1000, sms*128*2.0*clk*1e3/1e12);
  cudaError_t e=cudaGetLastError(); if(e) printf("err %s\n", cudaGetErrorString(e));
}
int main(){
  float *out,*in; cudaMalloc(&out, 148*32*256*4); cudaMalloc(&in, 4096*4);
  cudaMemset(in,0,4096*4);
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  int blocks=sms*8;
  run("ffma", k_ffma, 4.0*RV, 20000, blocks, out, in);
  run("ffma2", k_ffma2, 4.0*RV, 20000, blocks, out, in);
  run("smem_ffma", k_smem_ffma, 64.0*RV, 1250, blocks, out, in);
  run("smem_ffma2", k_smem_ffma2, 64.0*RV, 1250, blocks, out, in);
  return 0;
}
