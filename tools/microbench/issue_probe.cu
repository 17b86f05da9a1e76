// Cost of tm_tc_kernel's MMA issue pattern in isolation (one CTA per SM, one warp issuing, no
// producers): per stage (image row) 6 kind::f16 MMAs of M = 128, K = 16 -- (hi.hi, hi.lo, lo.hi)
// for each of the two K-steps of a 32-column chunk -- from a TMEM A buffer (6 buffers) and a B
// window of the reversed template block that moves by one 16-byte row per stage, accumulating
// into an N-column window of TMEM that moves by 8 columns per 8-stage group.  Mode bits remove
// one feature at a time:
//   1  no tcgen05.commit per stage (one per group)
//   2  B window start fixed (no per-stage row shift)
//   4  one A buffer (no rotation)
//   8  D window fixed at column 0
//  16  one thread issues (no elect / __syncwarp around the MMAs)
//  32  commit per stage, then wait for it before the next stage (latency of a stage; not with 1)
//  64  unrolled 6-MMA body (no wait / fence between the two K-steps)
// 128  B window start 128-byte aligned (row 8; with 2: fixed there, else 8 + 8 (s & 1))
// 256  LBO = 128 B x N / 8 (K halves packed back to back, as in the rate probes)
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -I../../paper_conf_ipps_moorelk13_b200/csrc -o issue_probe issue_probe.cu
#include <cstdio>
#include <cstdlib>
#include <vector>
#include "ncc_tc.cuh"

using namespace nccb;

__global__ void __launch_bounds__(128, 1) issue_kernel(int stages, int mode, int N, float* sink, long long* cyc) {
  extern __shared__ __align__(1024) unsigned char sm[];
  __shared__ __align__(8) uint64_t done[8], gdone;
  __shared__ uint32_t tbase_s;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  constexpr int kLB = tc::kLB;
  const uint32_t plane = kLB * 16;
  const int npl = 4;  // WC = 32: 4 planes of 8 bf16 per operand (hi, lo)
  for (int e = tid; e < 2 * npl * kLB * 4; e += blockDim.x) reinterpret_cast<uint32_t*>(sm)[e] = 0x3c003c00u + (e % 7);
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_u32(&tbase_s)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (tid == 0) {
    for (int b = 0; b < 8; ++b) mbar_init(&done[b], 1);
    mbar_init(&gdone, 1);
    fence_mbar_init();
  }
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const uint32_t tbase = tbase_s;
  {
    const uint32_t lb = (uint32_t)(warp * 32) << 16;
    uint32_t z[8];
    for (int k = 0; k < 8; ++k) z[k] = 0x3c003c00u;
    for (int c = 0; c < 512; c += 8) tc::st8(tbase + lb + c, z);
    tc::st_wait();
  }
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const long long t0 = clock64();
  if (warp == 0) {
    const uint32_t bhi = smem_u32(sm);
    const uint64_t dlo_off = (uint64_t)((npl * plane) >> 4);
    const uint64_t kKStep = (uint64_t)((2 * plane) >> 4);
    const uint32_t done0 = smem_u32(&done[0]);
    const bool leader = (mode & 16) ? lane == 0 : tc::elect_one();
    const uint32_t id = tc::idesc_bf16(N);
    int b = 0, ph = 0;
    for (int q = 0; q < stages; ++q) {
      const int g = q / 8, s = q % 8;
      const uint32_t col = (mode & 8) ? 0u : (uint32_t)((g * 8) % (320 - N - 8 > 0 ? (320 - N) / 8 * 8 : 8));
      const uint32_t dcol = tbase + col;
      const uint32_t lbo = (mode & 256) ? (uint32_t)N * 16 : plane;
      const uint64_t dg = tc::sdesc(bhi + (uint32_t)((mode & 128) ? 8 : 7) * 16, lbo, 128);
      const uint64_t dh = (mode & 128) ? dg + (uint64_t)((mode & 2) ? 0 : 8 * (s & 1)) : dg - (uint64_t)((mode & 2) ? 0 : s);
      const uint64_t dl = dh + dlo_off;
      const int bb = (mode & 4) ? 0 : b;
      const uint32_t ah = tbase + 320 + (uint32_t)(bb * 32), al = ah + 16;
      if ((mode & 16) ? lane == 0 : leader) {
        tc::mma_bf16(dcol, ah, dh, id);
        tc::mma_bf16(dcol, ah, dl, id);
        tc::mma_bf16(dcol, al, dh, id);
        if (mode & 64) {
          tc::mma_bf16(dcol, ah + 8, dh + kKStep, id);
          tc::mma_bf16(dcol, ah + 8, dl + kKStep, id);
          tc::mma_bf16(dcol, al + 8, dh + kKStep, id);
        }
      }
      if (!(mode & 16)) __syncwarp();
      if (!(mode & 64)) {
        tc::fence_after();
        if ((mode & 16) ? lane == 0 : leader) {
          tc::mma_bf16(dcol, ah + 8, dh + kKStep, id);
          tc::mma_bf16(dcol, ah + 8, dl + kKStep, id);
          tc::mma_bf16(dcol, al + 8, dh + kKStep, id);
        }
      }
      if ((mode & 16) ? lane == 0 : leader) {
        if (!(mode & 1) || s == 7) tc::commit_u32(done0 + 8 * b);
      }
      if (!(mode & 16)) __syncwarp();
      if ((mode & 32) && (!(mode & 1) || s == 7)) {
        tc::mbar_wait_u32(done0 + 8 * b, (uint32_t)ph);
        tc::fence_after();
      }
      if (++b == 6) {
        b = 0;
        ph ^= 1;
      }
    }
    if ((mode & 16) ? lane == 0 : leader) tc::commit_u32(smem_u32(&gdone));
    __syncwarp();
    tc::mbar_wait_u32(smem_u32(&gdone), 0u);
    tc::fence_after();
  }
  __syncthreads();
  if (tid == 0) cyc[blockIdx.x] = clock64() - t0;
  uint32_t v[8];
  tc::ld8(tbase + ((uint32_t)(warp * 32) << 16), v);
  if (v[0] == 12345u) sink[tid] = (float)v[1];
  tc::fence_before();
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tbase));
}

// Variants of umma_probe's rate_bf16_ts loop (one thread, D = column 0): which difference between
// that loop (45 cycles per MMA at N <= 80) and the kernel's pattern costs?
//   v 0  rate loop: 4 MMAs, A = 256 + 8 kk, B = K-step kk (LBO = 16 N), acc = (it | kk) > 0
//   v 1  as 0, accumulate always
//   v 2  as 0, tc::mma_bf16 ("memory" clobber, accumulate always)
//   v 3  6 MMAs per iteration: (A hi, B hi) (A hi, B lo) (A lo, B hi) for kk = 0, 1
//   v 4  as 3, A hi / lo = 256 + 8 kk / 272 + 8 kk and B hi / lo 2 K-steps apart (no operand repeats)
__device__ __forceinline__ void mma_acc(uint32_t d, uint32_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n\t}\n" ::"r"(d),
      "r"(a), "l"(b), "r"(idesc), "r"(acc));
}
__global__ void __launch_bounds__(128, 1) rate_var_kernel(int iters, int v, int N, float* sink, long long* cyc) {
  extern __shared__ __align__(1024) unsigned char sm[];
  __shared__ __align__(8) uint64_t bar;
  __shared__ uint32_t tbase_s;
  const int tid = threadIdx.x, warp = tid >> 5;
  for (int e = tid; e < 8 * N * 8; e += blockDim.x) reinterpret_cast<uint16_t*>(sm)[e] = (uint16_t)(0x3c00 + (e % 97));
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_u32(&tbase_s)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (tid == 0) {
    mbar_init(&bar, 1);
    fence_mbar_init();
  }
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const uint32_t d = tbase_s;
  {
    uint32_t z[8];
    for (int k = 0; k < 8; ++k) z[k] = 0x3c003c00u;
    for (int c = 0; c < 512; c += 8) tc::st8(d + ((uint32_t)(warp * 32) << 16) + c, z);
    tc::st_wait();
  }
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const long long t0 = clock64();
  const uint32_t id = tc::idesc_bf16(N), base = smem_u32(sm);
  int nm = 0;
  if (tid == 0) {
    for (int it = 0; it < iters; ++it) {
      if (v <= 2) {
        for (int kk = 0; kk < 4; ++kk) {
          const uint64_t b = tc::sdesc(base + kk * 2 * N * 16, N * 16, 128);
          if (v == 0) mma_acc(d, d + 256 + kk * 8, b, id, (it | kk) > 0);
          else if (v == 1) mma_acc(d, d + 256 + kk * 8, b, id, 1u);
          else tc::mma_bf16(d, d + 256 + kk * 8, b, id);
        }
        nm += 4;
      } else {
        for (int kk = 0; kk < 2; ++kk) {
          const uint64_t bh = tc::sdesc(base + kk * 2 * N * 16, N * 16, 128);
          const uint64_t bl = tc::sdesc(base + (kk + 2) * 2 * N * 16, N * 16, 128);
          const uint32_t ah = d + 256 + kk * 8, al = v == 3 ? d + 272 + kk * 8 : d + 272 + kk * 8;
          mma_acc(d, ah, bh, id, 1u);
          mma_acc(d, ah, v == 3 ? bl : bl, id, 1u);
          mma_acc(d, al, v == 3 ? bh : tc::sdesc(base + (kk + 1) * 2 * N * 16, N * 16, 128), id, 1u);
        }
        nm += 6;
      }
    }
    tc::commit(&bar);
  }
  __syncwarp();
  if (warp == 0) tc::mbar_wait_u32(smem_u32(&bar), 0u);
  __syncthreads();
  tc::fence_after();
  if (tid == 0) cyc[blockIdx.x] = (clock64() - t0) / (nm > 0 ? nm : 1);
  uint32_t vv[8];
  tc::ld8(d + ((uint32_t)(warp * 32) << 16), vv);
  if (vv[0] == 12345u) sink[tid] = (float)vv[1];
  tc::fence_before();
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(d));
}

// Starting from the fast straight-line loop (6 MMAs per iteration, loop-invariant operands: the
// pipe's rate), add the kernel's features one at a time (template bits, no run-time branching):
//   1 B window start moves back one 16-byte row per iteration (it % 8), LBO = the block's plane
//   2 A buffer rotates over 6 TMEM buffers (columns 320 + 32 b)
//   4 D window moves by 8 columns every 8 iterations
//   8 tcgen05.commit per iteration (to one of 6 mbarriers)
//  16 the whole warp runs the loop, the elected lane issues, __syncwarp per iteration
//  32 + a try_wait on an already completed mbarrier per iteration (whole warp)
//  64 + tcgen05.fence::after_thread_sync per iteration
template <int F>
__global__ void __launch_bounds__(640, 1) feat_kernel(int iters, int N, float* sink, long long* cyc) {
  extern __shared__ __align__(1024) unsigned char sm[];
  __shared__ __align__(8) uint64_t bar[8];
  __shared__ uint32_t tbase_s;
  const int tid = threadIdx.x, warp = tid >> 5;
  constexpr int kLB = tc::kLB;
  const uint32_t plane = kLB * 16;
  for (int e = tid; e < 8 * kLB * 4; e += blockDim.x) reinterpret_cast<uint32_t*>(sm)[e] = 0x3c003c00u + (e % 7);
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_u32(&tbase_s)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (tid == 0) {
    for (int b = 0; b < 8; ++b) mbar_init(&bar[b], 1);
    fence_mbar_init();
  }
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const uint32_t d = tbase_s;
  {
    uint32_t z[8];
    for (int k = 0; k < 8; ++k) z[k] = 0x3c003c00u;
    for (int c = 0; c < 512; c += 8) tc::st8(d + ((uint32_t)(warp * 32) << 16) + c, z);
    tc::st_wait();
  }
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const long long t0 = clock64();
  const uint32_t id = tc::idesc_bf16(N), base = smem_u32(sm);
  const uint32_t bar0 = smem_u32(&bar[0]);
  __shared__ __align__(8) uint64_t donebar;
  if (tid == 0) {
    mbar_init(&donebar, 1);
    fence_mbar_init();
    mbar_arrive(&donebar);  // phase 0 completes
  }
  __syncthreads();
  const bool leader = (F & 16) ? (warp == 0 && tc::elect_one()) : tid == 0;
  if ((F & 16) ? warp == 0 : tid == 0) {
    for (int it = 0; it < iters; ++it) {
      if (F & 32) {
        if (!tc::mbar_try_u32(smem_u32(&donebar), 0u)) tc::mbar_wait_u32(smem_u32(&donebar), 0u);
      }
      if (F & 64) tc::fence_after();
      const int s = (F & 1) ? (it & 7) : 0, b = (F & 2) ? it % 6 : 0;
      const uint32_t col = (F & 4) ? (uint32_t)(((it >> 3) * 8) % 176) : 0u;
      const uint64_t dg = tc::sdesc(base + 7 * 16, plane, 128) - (uint64_t)s;
      const uint64_t kst = (uint64_t)((2 * plane) >> 4), lo = (uint64_t)((4 * plane) >> 4);
      const uint32_t ah = d + 320 + (uint32_t)(b * 32), al = ah + 16, dc = d + col;
      if (leader) {
#pragma unroll
        for (int kk = 0; kk < 2; ++kk) {
          mma_acc(dc, ah + kk * 8, dg + kk * kst, id, 1u);
          mma_acc(dc, ah + kk * 8, dg + lo + kk * kst, id, 1u);
          mma_acc(dc, al + kk * 8, dg + kk * kst, id, 1u);
        }
        if (F & 8) tc::commit_u32(bar0 + 8 * b);
      }
      if (F & 16) __syncwarp();
    }
    if (leader) tc::commit_u32(bar0 + 8 * 7);
  }
  __syncwarp();
  if (warp == 0) tc::mbar_wait_u32(bar0 + 8 * 7, 0u);
  __syncthreads();
  tc::fence_after();
  if (tid == 0) cyc[blockIdx.x] = (clock64() - t0) / (6 * iters);
  uint32_t vv[8];
  tc::ld8(d + ((uint32_t)(warp * 32) << 16), vv);
  if (vv[0] == 12345u) sink[tid] = (float)vv[1];
  tc::fence_before();
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(d));
}
template <int F>
static void run_feat(int nsm, float* sink, long long* cyc, int N, int threads = 128, int smem = 8 * tc::kLB * 16 + 4096) {
  cudaFuncSetAttribute(feat_kernel<F>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  feat_kernel<F><<<nsm, threads, smem>>>(16, N, sink, cyc);
  feat_kernel<F><<<nsm, threads, smem>>>(2000, N, sink, cyc);
  cudaError_t e = cudaDeviceSynchronize();
  std::vector<long long> c(nsm);
  cudaMemcpy(c.data(), cyc, nsm * 8, cudaMemcpyDeviceToHost);
  double avg = 0;
  for (auto x : c) avg += x;
  printf("{\"feat\": %d, \"N\": %d, \"threads\": %d, \"smem\": %d, \"err\": \"%s\", \"cycles_per_mma\": %.1f}\n", F, N, threads, smem, cudaGetErrorString(e), avg / nsm);
}

int main(int argc, char** argv) {
  setvbuf(stdout, nullptr, _IONBF, 0);
  int nsm = 0;
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
  float* sink;
  long long* cyc;
  cudaMalloc(&sink, 4096);
  cudaMalloc(&cyc, nsm * 8);
  const int smem = 2 * 4 * tc::kLB * 16 + 4096;
  cudaFuncSetAttribute(issue_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  const int stages = 2048;
  const int modes[] = {0};
  const int Ns[] = {136};
  for (int N : Ns)
    for (int mode : modes) {
      issue_kernel<<<nsm, 128, smem>>>(16, mode, N, sink, cyc);
      issue_kernel<<<nsm, 128, smem>>>(stages, mode, N, sink, cyc);
      cudaError_t e = cudaDeviceSynchronize();
      std::vector<long long> c(nsm);
      cudaMemcpy(c.data(), cyc, nsm * 8, cudaMemcpyDeviceToHost);
      double avg = 0;
      for (auto x : c) avg += x;
      avg /= nsm;
      printf("{\"N\": %d, \"mode\": %d, \"err\": \"%s\", \"cycles_per_stage\": %.1f, \"cycles_per_mma\": %.1f}\n", N, mode,
             cudaGetErrorString(e), avg / stages, avg / stages / 6);
    }
  for (int N : {136, 64}) {
    run_feat<127>(nsm, sink, cyc, N, 640, 120 * 1024);
    run_feat<127>(nsm, sink, cyc, N, 640);
    run_feat<127>(nsm, sink, cyc, N, 128, 120 * 1024);
    run_feat<0>(nsm, sink, cyc, N);
    run_feat<1>(nsm, sink, cyc, N);
    run_feat<2>(nsm, sink, cyc, N);
    run_feat<4>(nsm, sink, cyc, N);
    run_feat<8>(nsm, sink, cyc, N);
    run_feat<15>(nsm, sink, cyc, N);
    run_feat<16>(nsm, sink, cyc, N);
    run_feat<16 | 32>(nsm, sink, cyc, N);
    run_feat<16 | 64>(nsm, sink, cyc, N);
    run_feat<16 | 32 | 64>(nsm, sink, cyc, N);
    run_feat<15 | 16 | 32 | 64>(nsm, sink, cyc, N);
    run_feat<32 | 64>(nsm, sink, cyc, N);
  }
  cudaFuncSetAttribute(rate_var_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 8 * 256 * 16);
  for (int N : {32, 80, 136})
    for (int v = 0; v < 5; ++v) {
      rate_var_kernel<<<nsm, 128, 8 * 256 * 16>>>(10, v, N, sink, cyc);
      rate_var_kernel<<<nsm, 128, 8 * 256 * 16>>>(2000, v, N, sink, cyc);
      cudaError_t e = cudaDeviceSynchronize();
      std::vector<long long> c(nsm);
      cudaMemcpy(c.data(), cyc, nsm * 8, cudaMemcpyDeviceToHost);
      double avg = 0;
      for (auto x : c) avg += x;
      printf("{\"rate_var\": %d, \"N\": %d, \"err\": \"%s\", \"cycles_per_mma\": %.1f}\n", v, N, cudaGetErrorString(e), avg / nsm);
    }
  return 0;
}
