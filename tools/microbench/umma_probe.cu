// tcgen05 kind::tf32 probe (sm_100a): validates the shared-memory descriptor / instruction
// descriptor encoding used by the tensor-core numerator (K-major, no swizzle, rows 16 B apart,
// operand windows starting at any row) against a host fp64 reference, and measures the MMA
// issue rate for M = 128 and several N (SS mode, optional concurrent st.shared traffic).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o umma_probe umma_probe.cu
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <cmath>
#include <vector>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { printf("CUDA %s at %s:%d\n", cudaGetErrorString(e_), __FILE__, __LINE__); exit(1); } } while (0)

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ uint64_t sdesc(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
  uint64_t d = 0;
  d |= (uint64_t)((saddr >> 4) & 0x3FFFu);
  d |= (uint64_t)((lbo >> 4) & 0x3FFFu) << 16;
  d |= (uint64_t)((sbo >> 4) & 0x3FFFu) << 32;
  d |= (uint64_t)1 << 46;  // descriptor version (sm_100)
  return d;                // base offset 0, SWIZZLE_NONE
}
__host__ __device__ constexpr uint32_t idesc_tf32(int M, int N) {
  return (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
}
__device__ __forceinline__ void mma_tf32(uint32_t d, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}\n" ::"r"(d),
      "l"(a), "l"(b), "r"(idesc), "r"(acc));
}
__device__ __forceinline__ void mma_commit(uint64_t* bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(su32(bar))
               : "memory");
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, int n) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su32(bar)), "r"(n));
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred P;\nW_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1;\n\t"
      "@!P bra W_%=;\n}" ::"r"(su32(bar)),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ bool elect_one() {
  uint32_t pred = 0;
  asm volatile("{\n\t.reg .pred P;\n\telect.sync _|P, 0xffffffff;\n\tselp.u32 %0, 1, 0, P;\n}" : "=r"(pred));
  return pred != 0;
}
__device__ __forceinline__ void fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void fence_async_smem() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }

template <int NCOL>
__device__ __forceinline__ void tmem_alloc(uint32_t* dst) {
  asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(su32(dst)), "n"(NCOL));
  asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
}
template <int NCOL>
__device__ __forceinline__ void tmem_free(uint32_t base) {
  asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(base), "n"(NCOL));
}
__device__ __forceinline__ void tmem_ld8(uint32_t addr, float* v) {
  uint32_t r[8];
  asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7])
               : "r"(addr));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
  for (int i = 0; i < 8; ++i) v[i] = __uint_as_float(r[i]);
}

// ---- correctness: D[128][N] = A[128][K] . Bwin[N][K]^T, Bwin = rows [s, s+N) of B[Lb][K]
template <int N, int K>
__global__ void probe_kernel(const float* A, const float* B, int Lb, int s, float* D) {
  extern __shared__ __align__(1024) unsigned char sm[];
  __shared__ uint64_t bar;
  __shared__ uint32_t tbase;
  float* As = reinterpret_cast<float*>(sm);           // [K/4 planes][128 rows][4]
  float* Bs = As + (K / 4) * 128 * 4;                 // [K/4 planes][Lb rows][4]
  const int tid = threadIdx.x, warp = tid >> 5;
  for (int e = tid; e < 128 * K; e += blockDim.x) {
    const int m = e / K, k = e % K;
    As[((k / 4) * 128 + m) * 4 + (k % 4)] = A[e];
  }
  for (int e = tid; e < Lb * K; e += blockDim.x) {
    const int n = e / K, k = e % K;
    Bs[((k / 4) * Lb + n) * 4 + (k % 4)] = B[e];
  }
  fence_async_smem();
  if (warp == 0) tmem_alloc<256>(&tbase);
  if (tid == 0) { mbar_init(&bar, 1); asm volatile("fence.mbarrier_init.release.cluster;"); }
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t d = tbase;
  if (tid == 0) {
    for (int kk = 0; kk < K / 8; ++kk) {
      const uint64_t a = sdesc(su32(As) + kk * 2 * 128 * 16, 128 * 16, 128);
      const uint64_t b = sdesc(su32(Bs) + kk * 2 * Lb * 16 + s * 16, Lb * 16, 128);
      mma_tf32(d, a, b, idesc_tf32(128, N), kk > 0);
    }
    mma_commit(&bar);
  }
  mbar_wait(&bar, 0);
  fence_after();
  const int lane_row = warp * 32 + (tid & 31);
  for (int c = 0; c < N; c += 8) {
    float v[8];
    tmem_ld8(d + ((uint32_t)(warp * 32) << 16) + c, v);
    for (int i = 0; i < 8; ++i) D[lane_row * N + c + i] = v[i];
  }
  fence_before();
  __syncthreads();
  if (warp == 0) tmem_free<256>(d);
}

// ---- throughput: ITERS x (K/8) MMAs of 128 x N x 8 on resident operands; optional st.shared
// traffic of `sts_bytes` per MMA from warps 1..3 (models the Hankel producer).
template <int N>
__global__ void rate_kernel(int iters, int sts_per_mma, float* sink, long long* cycles) {
  extern __shared__ __align__(1024) unsigned char sm[];
  __shared__ uint64_t bar;
  __shared__ uint32_t tbase;
  constexpr int K = 64;
  float* As = reinterpret_cast<float*>(sm);
  float* Bs = As + (K / 4) * 128 * 4;
  float* Ws = Bs + (K / 4) * N * 4;  // st.shared scratch, 32 KB
  const int tid = threadIdx.x, warp = tid >> 5;
  for (int e = tid; e < (K / 4) * 128 * 4 + (K / 4) * N * 4; e += blockDim.x) As[e] = 0.001f * (e % 97);
  fence_async_smem();
  if (warp == 0) tmem_alloc<256>(&tbase);
  if (tid == 0) { mbar_init(&bar, 1); asm volatile("fence.mbarrier_init.release.cluster;"); }
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t d = tbase;
  long long t0 = clock64();
  if (tid == 0) {
    for (int it = 0; it < iters; ++it)
      for (int kk = 0; kk < K / 8; ++kk) {
        const uint64_t a = sdesc(su32(As) + kk * 2 * 128 * 16, 128 * 16, 128);
        const uint64_t b = sdesc(su32(Bs) + kk * 2 * N * 16, N * 16, 128);
        mma_tf32(d, a, b, idesc_tf32(128, N), (it | kk) > 0);
      }
    mma_commit(&bar);
  } else if (warp >= 1 && sts_per_mma > 0) {
    // producers: st.shared.v4 traffic proportional to the MMA count (16 B per thread per store)
    const int t = tid - 32;
    const int nthr = blockDim.x - 32;
    const long long total = (long long)iters * (K / 8) * sts_per_mma / 16;
    float4 val = make_float4(1.f, 2.f, 3.f, 4.f);
    float4* w4 = reinterpret_cast<float4*>(Ws);
    for (long long e = t; e < total; e += nthr) {
      w4[e & 2047] = val;
      val.x += 1.0f;
    }
  }
  mbar_wait(&bar, 0);
  long long t1 = clock64();
  fence_after();
  if (tid == 0) cycles[blockIdx.x] = t1 - t0;
  float v[8];
  tmem_ld8(d + ((uint32_t)(warp * 32) << 16), v);
  if (v[0] == 12345.f) sink[tid] = v[1];
  fence_before();
  __syncthreads();
  if (warp == 0) tmem_free<256>(d);
}


__device__ __forceinline__ void mma_tf32_ts(uint32_t d, uint32_t a_tmem, uint64_t b, uint32_t idesc, uint32_t acc) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::tf32 [%0], [%1], %2, %3, p;\n\t}\n" ::"r"(d),
      "r"(a_tmem), "l"(b), "r"(idesc), "r"(acc));
}
__device__ __forceinline__ void tmem_st8(uint32_t addr, const float* v) {
  asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"r"(addr),
               "r"(__float_as_uint(v[0])), "r"(__float_as_uint(v[1])), "r"(__float_as_uint(v[2])),
               "r"(__float_as_uint(v[3])), "r"(__float_as_uint(v[4])), "r"(__float_as_uint(v[5])),
               "r"(__float_as_uint(v[6])), "r"(__float_as_uint(v[7]))
               : "memory");
}
__device__ __forceinline__ void tmem_st_wait() { asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory"); }

// ---- correctness, A from tensor memory: thread m writes row m of A into TMEM columns [256, 256+K)
template <int N, int K>
__global__ void probe_ts_kernel(const float* A, const float* B, int Lb, int s, float* D) {
  extern __shared__ __align__(1024) unsigned char sm[];
  __shared__ uint64_t bar;
  __shared__ uint32_t tbase;
  float* Bs = reinterpret_cast<float*>(sm);
  const int tid = threadIdx.x, warp = tid >> 5;
  for (int e = tid; e < Lb * K; e += blockDim.x) {
    const int n = e / K, k = e % K;
    Bs[((k / 4) * Lb + n) * 4 + (k % 4)] = B[e];
  }
  fence_async_smem();
  if (warp == 0) tmem_alloc<512>(&tbase);
  if (tid == 0) { mbar_init(&bar, 1); asm volatile("fence.mbarrier_init.release.cluster;"); }
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t d = tbase;
  const uint32_t lane_base = (uint32_t)(warp * 32) << 16;
  for (int c = 0; c < K; c += 8) tmem_st8(d + lane_base + 256 + c, A + tid * K + c);
  tmem_st_wait();
  fence_before();
  __syncthreads();
  fence_after();
  if (tid == 0) {
    for (int kk = 0; kk < K / 8; ++kk) {
      const uint64_t b = sdesc(su32(Bs) + kk * 2 * Lb * 16 + s * 16, Lb * 16, 128);
      mma_tf32_ts(d, d + 256 + kk * 8, b, idesc_tf32(128, N), kk > 0);
    }
    mma_commit(&bar);
  }
  mbar_wait(&bar, 0);
  fence_after();
  for (int c = 0; c < N; c += 8) {
    float v[8];
    tmem_ld8(d + lane_base + c, v);
    for (int i = 0; i < 8; ++i) D[tid * N + c + i] = v[i];
  }
  fence_before();
  __syncthreads();
  if (warp == 0) tmem_free<512>(d);
}

// ---- throughput, A from tensor memory (128 x 64 at column 256), B in shared memory
template <int N>
__global__ void rate_ts_kernel(int iters, float* sink, long long* cycles) {
  extern __shared__ __align__(1024) unsigned char sm[];
  __shared__ uint64_t bar;
  __shared__ uint32_t tbase;
  constexpr int K = 64;
  float* Bs = reinterpret_cast<float*>(sm);
  const int tid = threadIdx.x, warp = tid >> 5;
  for (int e = tid; e < (K / 4) * N * 4; e += blockDim.x) Bs[e] = 0.001f * (e % 97);
  fence_async_smem();
  if (warp == 0) tmem_alloc<512>(&tbase);
  if (tid == 0) { mbar_init(&bar, 1); asm volatile("fence.mbarrier_init.release.cluster;"); }
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t d = tbase;
  const uint32_t lane_base = (uint32_t)(warp * 32) << 16;
  float z[8] = {0.5f, 0.25f, 0.125f, 1.f, 2.f, 3.f, 4.f, 5.f};
  for (int c = 0; c < K; c += 8) tmem_st8(d + lane_base + 256 + c, z);
  tmem_st_wait();
  fence_before();
  __syncthreads();
  fence_after();
  long long t0 = clock64();
  if (tid == 0) {
    for (int it = 0; it < iters; ++it)
      for (int kk = 0; kk < K / 8; ++kk) {
        const uint64_t b = sdesc(su32(Bs) + kk * 2 * N * 16, N * 16, 128);
        mma_tf32_ts(d, d + 256 + kk * 8, b, idesc_tf32(128, N), (it | kk) > 0);
      }
    mma_commit(&bar);
  }
  mbar_wait(&bar, 0);
  long long t1 = clock64();
  fence_after();
  if (tid == 0) cycles[blockIdx.x] = t1 - t0;
  float v[8];
  tmem_ld8(d + lane_base, v);
  if (v[0] == 12345.f) sink[tid] = v[1];
  fence_before();
  __syncthreads();
  if (warp == 0) tmem_free<512>(d);
}

static float tf32r(float x) {  // round to nearest (ties away) at 10 mantissa bits
  uint32_t u;
  memcpy(&u, &x, 4);
  u = (u + 0x1000u) & 0xFFFFE000u;
  float y;
  memcpy(&y, &u, 4);
  return y;
}

template <int N, bool TS = false>
static int check(int s) {
  constexpr int K = 32;
  const int Lb = N + 24;
  std::vector<float> A(128 * K), B(Lb * K), D(128 * N);
  srand(1234 + N + s);
  for (auto& x : A) x = tf32r((float)rand() / RAND_MAX - 0.5f);
  for (auto& x : B) x = tf32r((float)rand() / RAND_MAX - 0.5f);
  float *dA, *dB, *dD;
  CK(cudaMalloc(&dA, A.size() * 4));
  CK(cudaMalloc(&dB, B.size() * 4));
  CK(cudaMalloc(&dD, D.size() * 4));
  CK(cudaMemcpy(dA, A.data(), A.size() * 4, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(dB, B.data(), B.size() * 4, cudaMemcpyHostToDevice));
  const int smem = (128 + Lb) * K * 4;
  if (TS) {
    CK(cudaFuncSetAttribute(probe_ts_kernel<N, K>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
    probe_ts_kernel<N, K><<<1, 128, smem>>>(dA, dB, Lb, s, dD);
  } else {
    CK(cudaFuncSetAttribute(probe_kernel<N, K>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
    probe_kernel<N, K><<<1, 128, smem>>>(dA, dB, Lb, s, dD);
  }
  CK(cudaGetLastError());
  CK(cudaDeviceSynchronize());
  CK(cudaMemcpy(D.data(), dD, D.size() * 4, cudaMemcpyDeviceToHost));
  double maxerr = 0.0;
  for (int m = 0; m < 128; ++m)
    for (int n = 0; n < N; ++n) {
      double r = 0.0;
      for (int k = 0; k < K; ++k) r += (double)A[m * K + k] * (double)B[(s + n) * K + k];
      maxerr = fmax(maxerr, fabs(r - D[m * N + n]));
    }
  printf("{\"probe\": \"%s\", \"N\": %d, \"s\": %d, \"max_abs_err\": %.3e, \"ok\": %s}\n", TS ? "tf32_ts" : "tf32_ss", N, s, maxerr,
         maxerr < 1e-4 ? "true" : "false");
  cudaFree(dA);
  cudaFree(dB);
  cudaFree(dD);
  return maxerr < 1e-4 ? 0 : 1;
}

template <int N>
static void rate(int sts_per_mma) {
  constexpr int K = 64;
  const int smem = (128 + N) * K * 4 + 32768;
  CK(cudaFuncSetAttribute(rate_kernel<N>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  float* sink;
  long long* cyc;
  int nsm = 0;
  CK(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0));
  CK(cudaMalloc(&sink, 4096));
  CK(cudaMalloc(&cyc, nsm * 8));
  const int iters = 2000;
  rate_kernel<N><<<nsm, 128, smem>>>(10, sts_per_mma, sink, cyc);
  CK(cudaDeviceSynchronize());
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaEventRecord(e0);
  rate_kernel<N><<<nsm, 128, smem>>>(iters, sts_per_mma, sink, cyc);
  cudaEventRecord(e1);
  CK(cudaDeviceSynchronize());
  float ms = 0;
  cudaEventElapsedTime(&ms, e0, e1);
  std::vector<long long> c(nsm);
  CK(cudaMemcpy(c.data(), cyc, nsm * 8, cudaMemcpyDeviceToHost));
  double avg = 0;
  for (auto x : c) avg += x;
  avg /= nsm;
  const double mmas = (double)iters * (K / 8);
  const double flops = 2.0 * 128 * N * 8 * mmas * nsm;
  printf("{\"probe\": \"rate\", \"N\": %d, \"sts_bytes_per_mma\": %d, \"cycles_per_mma\": %.2f, "
         "\"floor_cycles\": %.1f, \"tflops_tf32\": %.1f}\n",
         N, sts_per_mma, avg / mmas, 128.0 * N / 256.0, flops / (ms * 1e-3) / 1e12);
  cudaFree(sink);
  cudaFree(cyc);
}


template <int N>
static void rate_ts() {
  constexpr int K = 64;
  const int smem = N * K * 4;
  CK(cudaFuncSetAttribute(rate_ts_kernel<N>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  float* sink;
  long long* cyc;
  int nsm = 0;
  CK(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0));
  CK(cudaMalloc(&sink, 4096));
  CK(cudaMalloc(&cyc, nsm * 8));
  const int iters = 2000;
  rate_ts_kernel<N><<<nsm, 128, smem>>>(10, sink, cyc);
  CK(cudaDeviceSynchronize());
  rate_ts_kernel<N><<<nsm, 128, smem>>>(iters, sink, cyc);
  CK(cudaDeviceSynchronize());
  std::vector<long long> c(nsm);
  CK(cudaMemcpy(c.data(), cyc, nsm * 8, cudaMemcpyDeviceToHost));
  double avg = 0;
  for (auto x : c) avg += x;
  avg /= nsm;
  printf("{\"probe\": \"rate_ts\", \"N\": %d, \"cycles_per_mma\": %.2f, \"floor_cycles\": %.1f}\n", N,
         avg / ((double)iters * (K / 8)), 128.0 * N / 256.0);
  cudaFree(sink);
  cudaFree(cyc);
}

// ---- throughput variants (A in TMEM): B window offset (rows), D column offset, concurrent
// tcgen05.st traffic from warps 1..3 into spare TMEM columns, split of N into two MMAs.
template <int N>
__global__ void rate_ts2_kernel(int iters, int boff, int dcol, int sttm, int split, float* sink, long long* cycles) {
  extern __shared__ __align__(1024) unsigned char sm[];
  __shared__ uint64_t bar;
  __shared__ uint32_t tbase;
  __shared__ volatile int done;
  constexpr int K = 64;
  constexpr int LB = N + 16;
  float* Bs = reinterpret_cast<float*>(sm);
  const int tid = threadIdx.x, warp = tid >> 5;
  for (int e = tid; e < (K / 4) * LB * 4; e += blockDim.x) Bs[e] = 0.001f * (e % 97);
  fence_async_smem();
  if (warp == 0) tmem_alloc<512>(&tbase);
  if (tid == 0) { mbar_init(&bar, 1); asm volatile("fence.mbarrier_init.release.cluster;"); done = 0; }
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t d = tbase;
  const uint32_t lane_base = (uint32_t)(warp * 32) << 16;
  float z[8] = {0.5f, 0.25f, 0.125f, 1.f, 2.f, 3.f, 4.f, 5.f};
  for (int c = 0; c < K; c += 8) tmem_st8(d + lane_base + 320 + c, z);
  tmem_st_wait();
  fence_before();
  __syncthreads();
  fence_after();
  long long t0 = clock64();
  if (tid == 0) {
    for (int it = 0; it < iters; ++it)
      for (int kk = 0; kk < K / 8; ++kk) {
        const uint32_t bstart = su32(Bs) + kk * 2 * LB * 16 + boff * 16;
        if (split) {
          mma_tf32_ts(d + dcol, d + 320 + kk * 8, sdesc(bstart, LB * 16, 128), idesc_tf32(128, split), 1);
          mma_tf32_ts(d, d + 320 + kk * 8, sdesc(bstart + split * 16, LB * 16, 128), idesc_tf32(128, N - split), 1);
        } else {
          mma_tf32_ts(d + dcol, d + 320 + kk * 8, sdesc(bstart, LB * 16, 128), idesc_tf32(128, N), (it | kk) > 0);
        }
      }
    mma_commit(&bar);
    mbar_wait(&bar, 0);
    done = 1;
  } else if (warp >= 4 && sttm) {
    // warps 4..7 (lane quadrants 0..3) keep storing into columns [384, 448)
    int n = 0;
    while (!done) {
      for (int c = 0; c < 64; c += 8) tmem_st8(d + ((uint32_t)((warp & 3) * 32) << 16) + 384 + c, z);
      tmem_st_wait();
      ++n;
    }
    if (n == -1) sink[tid] = z[0];
  }
  if (tid == 0) cycles[blockIdx.x] = clock64() - t0;
  __syncthreads();
  fence_after();
  float v[8];
  tmem_ld8(d + ((uint32_t)((warp & 3) * 32) << 16), v);
  if (v[0] == 12345.f) sink[tid] = v[1];
  fence_before();
  __syncthreads();
  if (warp == 0) tmem_free<512>(d);
}

template <int N>
static void rate_ts2(int boff, int dcol, int sttm, int split, int smem_pad = 0) {
  constexpr int K = 64;
  const int smem = smem_pad ? smem_pad : (N + 16) * K * 4;
  CK(cudaFuncSetAttribute(rate_ts2_kernel<N>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  float* sink;
  long long* cyc;
  int nsm = 0;
  CK(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0));
  CK(cudaMalloc(&sink, 4096));
  CK(cudaMalloc(&cyc, nsm * 8));
  const int iters = 1000;
  rate_ts2_kernel<N><<<nsm, 256, smem>>>(10, boff, dcol, sttm, split, sink, cyc);
  CK(cudaDeviceSynchronize());
  rate_ts2_kernel<N><<<nsm, 256, smem>>>(iters, boff, dcol, sttm, split, sink, cyc);
  CK(cudaDeviceSynchronize());
  std::vector<long long> c(nsm);
  CK(cudaMemcpy(c.data(), cyc, nsm * 8, cudaMemcpyDeviceToHost));
  double avg = 0;
  for (auto x : c) avg += x;
  avg /= nsm;
  printf("{\"probe\": \"rate_ts2\", \"N\": %d, \"boff\": %d, \"dcol\": %d, \"sttm\": %d, \"split\": %d, \"cycles_per_step\": %.2f}\n",
         N, boff, dcol, sttm, split, avg / ((double)iters * (K / 8)));
  cudaFree(sink);
  cudaFree(cyc);
}

// ---- stage pattern of tm_tc_kernel: per stage 4 K-steps x 3 products (A hi/lo in TMEM, B hi/lo),
// then tcgen05.commit to a per-buffer mbarrier (commit_each = 0: one commit at the end).
__global__ void rate_stage_kernel(int stages, int commit_each, int wait_each, int flags, float* sink, long long* cycles) {
  extern __shared__ __align__(1024) unsigned char sm[];
  __shared__ uint64_t bar[4];
  __shared__ uint32_t tbase;
  constexpr int N = 136;
  const int LB = (flags & 32) ? 152 : 144;
  const uint32_t PL = LB * 16;
  float* Bs = reinterpret_cast<float*>(sm);
  const int tid = threadIdx.x, warp = tid >> 5;
  for (int e = tid; e < 2 * 8 * 152 * 4; e += blockDim.x) Bs[e] = 0.001f * (e % 97);
  fence_async_smem();
  if (warp == 0) tmem_alloc<512>(&tbase);
  if (tid == 0) { for (int b = 0; b < 4; ++b) mbar_init(&bar[b], 1); asm volatile("fence.mbarrier_init.release.cluster;"); }
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t d = tbase;
  const uint32_t bhi = su32(Bs), blo = bhi + 8 * PL;
  {
    float z[8] = {0.5f, 0.25f, 0.125f, 1.f, 2.f, 3.f, 4.f, 5.f};
    for (int c = 0; c < 512; c += 8) tmem_st8(d + ((uint32_t)(warp * 32) << 16) + c, z);
    tmem_st_wait();
    fence_before();
    __syncthreads();
    fence_after();
  }
  const int nk = (flags & 64) ? 8 : 4, np = (flags & 64) ? 1 : 3;
  long long t0 = clock64();
  if ((flags & 128) ? warp == 0 : tid == 0) {
    for (int q = 0; q < stages; ++q) {
      const int b = q & 3;
      const uint32_t col = (flags & 2) ? 0u : (uint32_t)(((q / 8) * 8) % 256);
      const uint32_t n1 = col + N <= 256 ? N : 256 - col;
      const uint32_t ab = (flags & 16) ? d + 320 : d + 256 + b * 64;
      for (int kk = 0; kk < nk; ++kk) {
        const uint32_t poff = (uint32_t)(2 * kk) * PL + (7 - (q & 7)) * 16;
        for (int p = 0; p < np; ++p) {
          const uint32_t at = ab + ((p == 2 && !(flags & 1)) ? 32 : 0) + kk * 8;
          const uint32_t bb = ((p == 1 && !(flags & 1)) ? blo : bhi) + ((flags & 4) ? (uint32_t)(2 * kk) * PL : poff);
          if (!(flags & 128) || elect_one()) {
            mma_tf32_ts(d + col, at, sdesc(bb, PL, 128), idesc_tf32(128, n1), 1);
            if (n1 < N) mma_tf32_ts(d, at, sdesc(bb + n1 * 16, PL, 128), idesc_tf32(128, N - n1), 1);
          }
          if (flags & 128) __syncwarp();
        }
      }
      if (commit_each && (!(flags & 128) || elect_one())) mma_commit(&bar[b]);
      if (flags & 128) __syncwarp();
    }
    if (!commit_each && (!(flags & 128) || elect_one())) mma_commit(&bar[0]);
    if (flags & 128) __syncwarp();
  }
  __syncthreads();
  if (tid == 0) {
    if (commit_each) { for (int q = stages - 4; q < stages; ++q) mbar_wait(&bar[q & 3], (q >> 2) & 1); }
    else mbar_wait(&bar[0], 0);
    cycles[blockIdx.x] = clock64() - t0;
  }
  __syncthreads();
  fence_after();
  float v[8];
  tmem_ld8(d + ((uint32_t)(warp * 32) << 16), v);
  if (v[0] == 12345.f) sink[tid] = v[1];
  fence_before();
  __syncthreads();
  if (warp == 0) tmem_free<512>(d);
}

static void rate_stage(int commit_each, int wait_each, int flags = 0, int smem_pad = 0) {
  const int smem = smem_pad ? smem_pad : 2 * 8 * 152 * 16;
  CK(cudaFuncSetAttribute(rate_stage_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  float* sink;
  long long* cyc;
  int nsm = 0;
  CK(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0));
  CK(cudaMalloc(&sink, 4096));
  CK(cudaMalloc(&cyc, nsm * 8));
  const int stages = 512;
  rate_stage_kernel<<<nsm, 128, smem>>>(stages, commit_each, wait_each, flags, sink, cyc);
  CK(cudaDeviceSynchronize());
  rate_stage_kernel<<<nsm, 128, smem>>>(stages, commit_each, wait_each, flags, sink, cyc);
  CK(cudaDeviceSynchronize());
  std::vector<long long> c(nsm);
  CK(cudaMemcpy(c.data(), cyc, nsm * 8, cudaMemcpyDeviceToHost));
  double avg = 0;
  for (auto x : c) avg += x;
  avg /= nsm;
  printf("{\"probe\": \"rate_stage\", \"commit_each\": %d, \"flags\": %d, \"smem\": %d, \"cycles_per_stage\": %.1f}\n",
         commit_each, flags, smem, avg / stages);
  cudaFree(sink);
  cudaFree(cyc);
}

// ---- copy of rate_ts2 with single mutations (mode bits): 1 commit per iteration, 2 always
// accumulate, 4 runtime (non-unrolled) K loop, 8 = loop body guarded by lane == 0 of warp 0
// with the rest of the CTA parked at __syncthreads.
__global__ void rate_mut_kernel(int iters, int mode, int nk_rt, float* sink, long long* cycles) {
  extern __shared__ __align__(1024) unsigned char sm[];
  __shared__ uint64_t bar[5];
  __shared__ uint32_t tbase;
  constexpr int K = 64, N = 136, LB = N + 16;
  float* Bs = reinterpret_cast<float*>(sm);
  const int tid = threadIdx.x, warp = tid >> 5;
  for (int e = tid; e < 2 * (K / 4) * LB * 4; e += blockDim.x) Bs[e] = 0.001f * (e % 97);
  fence_async_smem();
  if (warp == 0) tmem_alloc<512>(&tbase);
  if (tid == 0) { for (int b = 0; b < 5; ++b) mbar_init(&bar[b], 1); asm volatile("fence.mbarrier_init.release.cluster;"); }
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t d = tbase;
  const uint32_t lane_base = (uint32_t)(warp * 32) << 16;
  float z[8] = {0.5f, 0.25f, 0.125f, 1.f, 2.f, 3.f, 4.f, 5.f};
  if (warp < 4) for (int c = 0; c < K; c += 8) tmem_st8(d + lane_base + 320 + c, z);
  tmem_st_wait();
  fence_before();
  __syncthreads();
  fence_after();
  long long t0 = clock64();
  const int issuer = (mode & 128) ? 12 * 32 : 0;
  if (tid == issuer) {
    for (int it = 0; it < iters; ++it) {
      if (mode & 4) {
        for (int kk = 0; kk < nk_rt; ++kk) {
          const uint64_t b = sdesc(su32(Bs) + kk * 2 * LB * 16, LB * 16, 128);
          mma_tf32_ts(d, d + 320 + kk * 8, b, idesc_tf32(128, N), (mode & 2) ? 1 : ((it | kk) > 0));
        }
      } else {
#pragma unroll
        for (int kk = 0; kk < K / 8; ++kk) {
          const int kb = (mode & 64) ? (kk % 4) : kk;            // 3-product pattern: 4 K-steps x 3
          const int pp = (mode & 64) ? (kk / 4) % 3 : 0;
          const uint32_t boff = ((mode & 16) && (kk & 1)) || ((mode & 64) && pp == 1) ? (uint32_t)(8 * LB * 16) : 0u;
          const uint32_t aoff = ((mode & 32) && (kk & 1)) || ((mode & 64) && pp == 2) ? 32u : 0u;
          const uint64_t b = sdesc(su32(Bs) + kb * 2 * LB * 16 + boff, LB * 16, 128);
          mma_tf32_ts(d, d + 320 + kb * 8 + aoff, b, idesc_tf32(128, N), (mode & 2) ? 1 : ((it | kk) > 0));
        }
      }
      if (mode & 1) mma_commit(&bar[it & 3]);
    }
    mma_commit(&bar[4]);
    if (!(mode & 8)) {
      mbar_wait(&bar[4], 0);
      cycles[blockIdx.x] = clock64() - t0;
    }
  }
  if (mode & 8) {
    __syncthreads();
    if (tid == issuer) {
      mbar_wait(&bar[4], 0);
      cycles[blockIdx.x] = clock64() - t0;
    }
  } else {
    mbar_wait(&bar[4], 0);
  }
  __syncthreads();
  fence_after();
  float v[8];
  tmem_ld8(d + ((uint32_t)((warp & 3) * 32) << 16), v);
  if (v[0] == 12345.f) sink[tid] = v[1];
  fence_before();
  __syncthreads();
  if (warp == 0) tmem_free<512>(d);
}

static void rate_mut(int mode, int threads = 256) {
  const int smem = 150000;
  CK(cudaFuncSetAttribute(rate_mut_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  float* sink;
  long long* cyc;
  int nsm = 0;
  CK(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0));
  CK(cudaMalloc(&sink, 4096));
  CK(cudaMalloc(&cyc, nsm * 8));
  const int iters = 1000;
  rate_mut_kernel<<<nsm, threads, smem>>>(10, mode, 8, sink, cyc);
  CK(cudaDeviceSynchronize());
  rate_mut_kernel<<<nsm, threads, smem>>>(iters, mode, 8, sink, cyc);
  CK(cudaDeviceSynchronize());
  std::vector<long long> c(nsm);
  CK(cudaMemcpy(c.data(), cyc, nsm * 8, cudaMemcpyDeviceToHost));
  double avg = 0;
  for (auto x : c) avg += x;
  avg /= nsm;
  printf("{\"probe\": \"rate_mut\", \"mode\": %d, \"threads\": %d, \"cycles_per_mma\": %.2f}\n", mode, threads,
         avg / (iters * 8.0));
  cudaFree(sink);
  cudaFree(cyc);
}

// ---- replica of tm_tc_kernel's MMA stream (no producers): per stage 4 K-steps x 3 products,
// B window start row 7 - (q % 8), D window start (8 * (q / 8)) % 192, A buffer q % 3; whole warp
// runs the loop, one elected lane issues.  mode bits: 1 fixed B start, 2 fixed D, 4 fixed A buf.
__global__ void rate_k_kernel(int stages, int mode, float* sink, long long* cycles) {
  extern __shared__ __align__(1024) unsigned char sm[];
  __shared__ uint64_t bar[4];
  __shared__ uint32_t tbase;
  constexpr int NW = 136, LB = 144;
  constexpr uint32_t PL = LB * 16;
  const int tid = threadIdx.x, warp = tid >> 5;
  float* Bs = reinterpret_cast<float*>(sm);
  for (int e = tid; e < 2 * 8 * LB * 4; e += blockDim.x) Bs[e] = (mode & 16) ? 0.0f : 0.001f * (e % 97);
  fence_async_smem();
  if (warp == 0) tmem_alloc<512>(&tbase);
  if (tid == 0) {
    for (int b = 0; b < 4; ++b) mbar_init(&bar[b], 1);
    asm volatile("fence.mbarrier_init.release.cluster;");
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(su32(&bar[3])) : "memory");
  }
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t d = tbase;
  {
    float z[8] = {0.5f, 0.25f, 0.125f, 1.f, 2.f, 3.f, 4.f, 5.f};
    if (mode & 16) for (int k = 0; k < 8; ++k) z[k] = 0.0f;
    if (warp < 4) for (int c = 0; c < 512; c += 8) tmem_st8(d + ((uint32_t)(warp * 32) << 16) + c, z);
    tmem_st_wait();
    fence_before();
    __syncthreads();
    fence_after();
  }
  long long t0 = clock64();
  if (tid == 0) sink[4000] = 0.0f;
  __syncthreads();
  if (warp == 0) {
    const uint32_t bhi = su32(Bs);
    const uint64_t dlo_off = (uint64_t)((8 * PL) >> 4);
    constexpr uint64_t kKStep = (uint64_t)((2 * PL) >> 4);
    int b = 0;
    for (int q = 0; q < stages; ++q) {
      const int s = (mode & 1) ? 0 : (q & 7), g = (mode & 2) ? 0 : q >> 3;
      const uint32_t col = (uint32_t)((g * 8) % 192);
      const uint64_t dh = sdesc(bhi + (uint32_t)(7 - s) * 16, PL, 128);
      const uint64_t dl = dh + dlo_off;
      const uint32_t ah = d + 320 + (uint32_t)(((mode & 4) ? 0 : b) * 64), al = ah + 32;
      const uint32_t dcol = d + col;
      if (elect_one()) {
        const uint32_t id = idesc_tf32(128, NW);
#pragma unroll
        for (int kk = 0; kk < 4; ++kk) {
          mma_tf32_ts(dcol, ah + kk * 8, dh + kk * kKStep, id, 1);
          mma_tf32_ts(dcol, ah + kk * 8, dl + kk * kKStep, id, 1);
          mma_tf32_ts(dcol, al + kk * 8, dh + kk * kKStep, id, 1);
        }
        mma_commit(&bar[b]);
      }
      __syncwarp();
      if ((mode & 8) && (tid & 31) == 0 && q < 1024) { sink[1024 + q] = (float)clock64(); }
      if (mode & 32) mbar_wait(&bar[3], 0);  // an already-completed barrier phase
      if (mode & 64) fence_after();
      if (mode & 512) {  // per-stage issue gap of ((mode >> 20) & 255) * 50 cycles
        const long long t1 = clock64();
        while (clock64() - t1 < (long long)((mode >> 20) & 255) * 50) {
        }
      }
      if (++b == 3) b = 0;
    }
    if (tid == 0) {
      const int ql = stages - 1;
      mbar_wait(&bar[ql % 3], (ql / 3) & 1);
      cycles[blockIdx.x] = clock64() - t0;
      *(volatile int*)&sink[4000] = 1;  // stop flag for the busy warps
      if (mode & 32768) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(su32(&bar[2])) : "memory");
    }
    if (mode & 65536) asm volatile("bar.arrive 1, %0;" ::"r"((int)blockDim.x - 128 + 32) : "memory");
  } else if ((mode & (4096 | 8192)) && warp >= 4 && (((mode & 4096) && (warp & 3) == 0) || ((mode & 8192) && (warp & 3) != 0))) {
    // spinning waiters: mbarrier try_wait on a phase that completes only at the end (bar[2])
    for (long long it = 0; it < (1ll << 28); ++it) {
      uint32_t done = 0;
      asm volatile(
          "{\n\t.reg .pred P;\n\tmbarrier.try_wait.parity.shared::cta.b64 P, [%1], %2;\n\tselp.u32 %0, 1, 0, P;\n}"
          : "=r"(done)
          : "r"(su32(&bar[2])), "r"(0u)
          : "memory");
      if (done || *(volatile int*)&sink[4000]) break;
      if (mode & 16384) __nanosleep(200);
    }
  } else if ((mode & 32768) && warp >= 4) {
    // waiters with a long suspend-time hint (the thread sleeps in the barrier until the phase completes)
    for (long long it = 0; it < (1ll << 20); ++it) {
      uint32_t done = 0;
      asm volatile(
          "{\n\t.reg .pred P;\n\tmbarrier.try_wait.parity.shared::cta.b64 P, [%1], %2, %3;\n\tselp.u32 %0, 1, 0, P;\n}"
          : "=r"(done)
          : "r"(su32(&bar[2])), "r"(0u), "r"(1000000u)
          : "memory");
      if (done) break;
    }
  } else if ((mode & 65536) && warp >= 4) {
    // waiters blocked on a named hardware barrier (released by the MMA thread at the end)
    asm volatile("bar.sync 1, %0;" ::"r"((int)blockDim.x - 128 + 32) : "memory");
  } else if ((mode & 128) && warp >= 4 && (!(mode & 1024) || (warp & 3) != 0) && (!(mode & 2048) || (warp & 3) == 0)) {
    // busy warps: dependent-free FMA stream with a sleep duty cycle (mode >> 8: sleep ns per 64 FMAs)
    float a0 = tid, a1 = tid + 1, a2 = tid + 2, a3 = tid + 3;
    const int sl = (mode & (1024 | 2048)) ? 0 : (mode >> 8);
    for (int it = 0; it < 200000; ++it) {
#pragma unroll
      for (int k = 0; k < 16; ++k) {
        a0 = fmaf(a0, 1.0001f, 0.5f); a1 = fmaf(a1, 1.0001f, 0.5f); a2 = fmaf(a2, 1.0001f, 0.5f); a3 = fmaf(a3, 1.0001f, 0.5f);
      }
      if (sl) __nanosleep(sl);
      if ((it & 63) == 0 && *(volatile int*)&sink[4000]) break;
    }
    if (a0 + a1 + a2 + a3 == 1.2345f) sink[tid] = a0;
  }
  __syncthreads();
  fence_after();
  float v[8];
  tmem_ld8(d + ((uint32_t)((warp & 3) * 32) << 16), v);
  if (v[0] == 12345.f) sink[tid] = v[1];
  fence_before();
  __syncthreads();
  if (warp == 0) tmem_free<512>(d);
}

static void rate_k(int mode, int threads = 128, int smem = 150000) {
  CK(cudaFuncSetAttribute(rate_k_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  float* sink;
  long long* cyc;
  int nsm = 0;
  CK(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0));
  CK(cudaMalloc(&sink, 65536));
  CK(cudaMalloc(&cyc, nsm * 8));
  const int stages = 600;
  rate_k_kernel<<<nsm, threads, smem>>>(30, mode, sink, cyc);
  CK(cudaDeviceSynchronize());
  rate_k_kernel<<<nsm, threads, smem>>>(stages, mode, sink, cyc);
  CK(cudaDeviceSynchronize());
  std::vector<long long> c(nsm);
  CK(cudaMemcpy(c.data(), cyc, nsm * 8, cudaMemcpyDeviceToHost));
  double avg = 0;
  for (auto x : c) avg += x;
  avg /= nsm;
  printf("{\"probe\": \"rate_k\", \"mode\": %d, \"threads\": %d, \"smem\": %d, \"cycles_per_stage\": %.1f, \"per_mma\": %.1f}\n", mode, threads, smem, avg / stages,
         avg / stages / 12);
  cudaFree(sink);
  cudaFree(cyc);
}


// ---- bf16 (kind::f16) M=128 K=16 MMA rate with A in TMEM: 2 bf16 per 32-bit TMEM column
__host__ __device__ constexpr uint32_t idesc_bf16(int M, int N) {
  return (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
}
__device__ __forceinline__ void mma_f16_ts(uint32_t d, uint32_t a_tmem, uint64_t b, uint32_t idesc, uint32_t acc) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n\t}\n" ::"r"(d),
      "r"(a_tmem), "l"(b), "r"(idesc), "r"(acc));
}
template <int N>
__global__ void rate_bf16_ts_kernel(int iters, float* sink, long long* cycles) {
  extern __shared__ __align__(1024) unsigned char sm[];
  __shared__ uint64_t bar;
  __shared__ uint32_t tbase;
  constexpr int K = 64;  // bf16 elements
  uint16_t* Bs = reinterpret_cast<uint16_t*>(sm);
  const int tid = threadIdx.x, warp = tid >> 5;
  for (int e = tid; e < (K / 8) * N * 8; e += blockDim.x) Bs[e] = (uint16_t)(0x3c00 + (e % 97));
  fence_async_smem();
  if (warp == 0) tmem_alloc<512>(&tbase);
  if (tid == 0) { mbar_init(&bar, 1); asm volatile("fence.mbarrier_init.release.cluster;"); }
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t d = tbase;
  const uint32_t lane_base = (uint32_t)(warp * 32) << 16;
  float z[8] = {0.5f, 0.25f, 0.125f, 1.f, 2.f, 3.f, 4.f, 5.f};
  for (int c = 0; c < K / 2; c += 8) tmem_st8(d + lane_base + 256 + c, z);
  tmem_st_wait();
  fence_before();
  __syncthreads();
  fence_after();
  long long t0 = clock64();
  if (tid == 0) {
    for (int it = 0; it < iters; ++it)
      for (int kk = 0; kk < K / 16; ++kk) {
        const uint64_t b = sdesc(su32(Bs) + kk * 2 * N * 16, N * 16, 128);
        mma_f16_ts(d, d + 256 + kk * 8, b, idesc_bf16(128, N), (it | kk) > 0);
      }
    mma_commit(&bar);
  }
  mbar_wait(&bar, 0);
  long long t1 = clock64();
  fence_after();
  if (tid == 0) cycles[blockIdx.x] = t1 - t0;
  float v[8];
  tmem_ld8(d + lane_base, v);
  if (v[0] == 12345.f) sink[tid] = v[1];
  fence_before();
  __syncthreads();
  if (warp == 0) tmem_free<512>(d);
}
template <int N>
static void rate_bf16_ts() {
  constexpr int K = 64;
  const int smem = N * K * 2;
  CK(cudaFuncSetAttribute(rate_bf16_ts_kernel<N>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  float* sink;
  long long* cyc;
  int nsm = 0;
  CK(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0));
  CK(cudaMalloc(&sink, 4096));
  CK(cudaMalloc(&cyc, nsm * 8));
  const int iters = 2000;
  rate_bf16_ts_kernel<N><<<nsm, 128, smem>>>(10, sink, cyc);
  CK(cudaDeviceSynchronize());
  rate_bf16_ts_kernel<N><<<nsm, 128, smem>>>(iters, sink, cyc);
  CK(cudaDeviceSynchronize());
  std::vector<long long> c(nsm);
  CK(cudaMemcpy(c.data(), cyc, nsm * 8, cudaMemcpyDeviceToHost));
  double avg = 0;
  for (auto x : c) avg += x;
  avg /= nsm;
  printf("{\"probe\": \"rate_bf16_ts\", \"N\": %d, \"cycles_per_mma\": %.2f, \"floor_cycles\": %.1f}\n", N,
         avg / ((double)iters * (K / 16)), 128.0 * N / 256.0);
  cudaFree(sink);
  cudaFree(cyc);
}

int main(int argc, char** argv) {
  setvbuf(stdout, nullptr, _IONBF, 0);
  if (argc > 1 && strcmp(argv[1], "rates") == 0) {  // cycles per M=128 K=8 tf32 MMA vs N, A from smem / TMEM
    rate<16>(0); rate<32>(0); rate<48>(0); rate<64>(0); rate<80>(0); rate<136>(0); rate<256>(0);
    rate_ts<16>(); rate_ts<32>(); rate_ts<48>(); rate_ts<64>(); rate_ts<80>(); rate_ts<136>(); rate_ts<256>();
    rate_bf16_ts<16>(); rate_bf16_ts<32>(); rate_bf16_ts<48>(); rate_bf16_ts<64>(); rate_bf16_ts<80>();
    rate_bf16_ts<136>(); rate_bf16_ts<256>();
    return 0;
  }
  rate_k(0, 576, 125000);
  rate_k(128, 576, 125000);
  rate_k(128 | 1024, 576, 125000);  // busy warps only on the other three SMSPs
  rate_k(128 | 2048, 576, 125000);  // busy warps only on the MMA warp's SMSP
  rate_k(4096, 576, 125000);        // try_wait spinners on the MMA warp's SMSP (warps 4, 8, 12, 16)
  rate_k(4096, 160, 125000);        // one spinner on the MMA warp's SMSP (warp 4)
  rate_k(8192, 576, 125000);        // spinners on the other SMSPs
  rate_k(4096 | 16384, 576, 125000);  // spinners with nanosleep(200) on the MMA warp's SMSP
  rate_k(32768, 576, 125000);       // waiters with a long try_wait suspend-time hint
  rate_k(65536, 576, 125000);       // waiters blocked in bar.sync
  return 0;
}
