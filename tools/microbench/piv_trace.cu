// Per-stage timeline of piv_ws2_kernel (CTA 0) on cfg3 / cfg4 shapes: clock64 stamps of
// producer thread 0 (loop start, after the empty wait, after the mask statistics, full arrival,
// search regions landed, border done, epilogue start / end) and consumer thread 0 (core start,
// core end, after the score-tile wait).  Random frames, constant window sums (timing only).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -DNCC_PIV_TRACE
//     -I../../paper_conf_ipps_moorelk13_b200/csrc -o piv_trace piv_trace.cu -lcuda
// usage: piv_trace <3|4> [pairs] [experiment bits: 1 no border sums, 2 no epilogue normalisation]
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <cuda.h>
#include "ncc_kernels.cuh"

using namespace nccb;

template <int TH, int TW, int MY, int MX, int CW, int WPS>
int run(int H, int W, int S, int P) {
  using Sh = PivWs2Shape<TH, TW, MY, MX, 16, CW, WPS>;
  auto kern = piv_ws2_kernel<TH, TW, MY, MX, 16, CW, 8, 8, WPS>;
  const int Ky = (H - TH - 2 * MY) / S + 1, Kx = (W - TW - 2 * MX) / S + 1;
  const int mh = H - TH + 1, mw = W - TW + 1;
  float *A, *B;
  double *S1, *S2;
  VecOut* vec;
  long long* tr;
  const size_t fe = (size_t)H * W;
  cudaMalloc(&A, fe * P * 4);
  cudaMalloc(&B, fe * P * 4);
  std::vector<float> hf(fe * P);
  srand(1);
  for (auto& x : hf) x = (float)rand() / RAND_MAX;
  cudaMemcpy(A, hf.data(), fe * P * 4, cudaMemcpyHostToDevice);
  cudaMemcpy(B, hf.data(), fe * P * 4, cudaMemcpyHostToDevice);
  cudaMalloc(&S1, (size_t)mh * mw * P * 8);
  cudaMalloc(&S2, (size_t)mh * mw * P * 8);
  std::vector<double> s1((size_t)mh * mw * P, 0.5 * TH * TW), s2((size_t)mh * mw * P, 0.4 * TH * TW);
  cudaMemcpy(S1, s1.data(), s1.size() * 8, cudaMemcpyHostToDevice);
  cudaMemcpy(S2, s2.data(), s2.size() * 8, cudaMemcpyHostToDevice);
  cudaMalloc(&vec, (size_t)P * Ky * Kx * sizeof(VecOut));
  cudaMalloc(&tr, 16 * 64 * 8);
  cudaMemset(tr, 0, 16 * 64 * 8);
  cudaMemcpyToSymbol(g_piv_trace, &tr, sizeof(tr));
  PivArgs a{};
  a.A = A; a.B = B; a.pitch = W; a.frame_stride = (int64_t)fe;
  a.H = H; a.W = W; a.h = TH; a.w = TW; a.my = MY; a.mx = MX; a.sy = S; a.sx = S; a.Ky = Ky; a.Kx = Kx;
  a.pair0 = 0; a.S1 = S1; a.S2 = S2; a.map_pitch = mw; a.map_frame_stride = (int64_t)mh * mw;
  a.vec = vec; a.scores = nullptr; a.subpix = 0; a.BP = Sh::BP; a.ssd = 0;
  CUtensorMap map;
  cuuint64_t gd[3] = {(cuuint64_t)W, (cuuint64_t)H, (cuuint64_t)P}, gs[2] = {(cuuint64_t)W * 4, (cuuint64_t)fe * 4};
  cuuint32_t bx[3] = {(cuuint32_t)Sh::BP, (cuuint32_t)(TH + 2 * MY), 1}, es[3] = {1, 1, 1};
  CUresult cr = cuTensorMapEncodeTiled(&map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3, B, gd, gs, bx, es,
                                       CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                                       CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (cr != CUDA_SUCCESS) { printf("encode failed %d\n", (int)cr); return 1; }
  cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, Sh::smem_bytes);
  int nsm = 0;
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
  const int total = P * Ky * Kx, ngroups = (total + WPS - 1) / WPS, grid = ngroups < nsm ? ngroups : nsm;
  float* flush;
  cudaMalloc(&flush, 512 << 20);
  for (int it = 0; it < 3; ++it) kern<<<grid, 16 * 32, Sh::smem_bytes>>>(a, map, total);
  cudaMemset(flush, 0, 512 << 20);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0); cudaEventCreate(&e1);
  cudaEventRecord(e0);
  kern<<<grid, 16 * 32, Sh::smem_bytes>>>(a, map, total);
  cudaEventRecord(e1);
  cudaError_t e = cudaDeviceSynchronize();
  float ms = 0; cudaEventElapsedTime(&ms, e0, e1);
  printf("kernel %.3f ms (%s), grid %d, groups %d, stages of CTA0 %d\n", ms, cudaGetErrorString(e), grid, ngroups,
         (ngroups + grid - 1) / grid);
  std::vector<long long> h(16 * 64);
  cudaMemcpy(h.data(), tr, h.size() * 8, cudaMemcpyDeviceToHost);
  long long t0 = h[0];
  for (int k = 0; k < 64; ++k) t0 = (h[8 * 64 + k] && h[8 * 64 + k] < t0) ? h[8 * 64 + k] : t0;
  const char* names[11] = {"P.start", "P.empty", "P.stats", "P.full", "P.landed", "P.border", "P.epi0", "P.epi1",
                           "C.core0", "C.core1", "C.scwait"};
  printf("stage");
  for (int sl = 0; sl < 11; ++sl) printf(" %9s", names[sl]);
  printf("\n");
  const int ns = (ngroups + grid - 1) / grid;
  for (int k = 0; k < ns && k < 64; ++k) {
    printf("%5d", k);
    for (int sl = 0; sl < 11; ++sl) printf(" %9lld", h[sl * 64 + k] ? h[sl * 64 + k] - t0 : -1ll);
    printf("\n");
  }
  return 0;
}

int main(int argc, char** argv) {
  const int cfg = argc > 1 ? atoi(argv[1]) : 3;
  const int P = argc > 2 ? atoi(argv[2]) : 1;
  const int exp = argc > 3 ? atoi(argv[3]) : 0;
  cudaMemcpyToSymbol(g_piv_exp, &exp, sizeof(exp));
  if (cfg == 3) return run<32, 32, 16, 16, 32, 4>(1024, 1024, 16, P);
  return run<64, 64, 32, 32, 64, 1>(2048, 2048, 32, P);
}
