// Per-stage timeline of tm_tc_kernel (CTA 0) on a cfg2-shaped problem (1024^2 image, 128^2
// template, WC = 32, 4 segments): clock64 stamps of the producer (after the mma_done wait,
// after the bf16 permutes, after the TMEM stores) and of the MMA issuer (after the a_full wait,
// after the commit).  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -DNCC_TC_TRACE
//   -I../../paper_conf_ipps_moorelk13_b200/csrc -o tc_trace tc_trace.cu -lcuda
#include <cstdio>
#include <vector>
#include <cuda.h>
#include "ncc_tc.cuh"

int main(int argc, char** argv) {
  using namespace nccb;
  const int H = 1024, W = 1024, h = 128, w = 128, U = H - h + 1, V = W - w + 1;
  const int WC = argc > 1 ? atoi(argv[1]) : 32, nseg = argc > 2 ? atoi(argv[2]) : 4;
  const int exp = argc > 3 ? atoi(argv[3]) : 0;
  cudaMemcpyToSymbol(g_tc_exp, &exp, sizeof(exp));
  const int nbi = 1, nbj = (w + WC - 1) / WC, vtiles = (V + 127) / 128;
  float *img, *tcB, *part;
  long long* tr;
  cudaMalloc(&img, (size_t)H * W * 16);  // two planes of 8-byte pair elements per row (tm_tc_split)
  cudaMemset(img, 0, (size_t)H * W * 16);
  cudaMalloc(&tcB, (size_t)nbi * nbj * tc::b_bytes(WC));
  cudaMemset(tcB, 0, (size_t)nbi * nbj * tc::b_bytes(WC));
  cudaMalloc(&part, (size_t)U * V * 4);
  cudaMalloc(&tr, 8 * 1024 * 8);
  cudaMemset(tr, 0, 8 * 1024 * 8);
  cudaMemcpyToSymbol(g_tc_trace, &tr, sizeof(tr));
  TcArgs a{};
  a.H = H; a.W = W;
  a.tcB = tcB; a.WC = WC; a.nbi = nbi; a.nbj = nbj; a.V = V; a.u_begin = 0; a.u_end = U;
  a.useg = (U + nseg - 1) / nseg; a.nseg = nseg; a.vtiles = vtiles; a.acc = part;
  a.acc_frame_stride = (int64_t)U * V;
  // chain / epilogue scratch (zero statistics: the normalised values are not inspected here)
  const int ngrp = (a.useg + tc::kHB - 1 + tc::kG - 1) / tc::kG;
  unsigned int* flags; unsigned long long *ticket, *keys; double* S; TemplateStats* ts;
  cudaMalloc(&flags, (size_t)vtiles * nseg * ngrp * 4 * 4); cudaMemset(flags, 0, (size_t)vtiles * nseg * ngrp * 16);
  cudaMalloc(&ticket, 8); cudaMemset(ticket, 0, 8);
  cudaMalloc(&keys, 8); cudaMemset(keys, 0, 8);
  cudaMalloc(&S, (size_t)U * V * 8); cudaMemset(S, 0, (size_t)U * V * 8);
  cudaMalloc(&ts, sizeof(TemplateStats)); cudaMemset(ts, 0, sizeof(TemplateStats));
  float* fz;
  cudaMalloc(&fz, (size_t)U * V * 4); cudaMemset(fz, 0, (size_t)U * V * 4);
  a.rsv = fz; a.mean = fz;
  a.flags = flags; a.ngrp_max = ngrp; a.ticket = ticket; a.S1 = S; a.S2 = S; a.stat_frame_stride = (int64_t)U * V;
  a.tst = ts; a.h = h; a.w = w; a.scores = nullptr; a.score_frame_stride = 0; a.keys = keys; a.ssd = 0;
  const int smem = tc::smem_bytes(WC);
  cudaFuncSetAttribute(tm_tc_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  dim3 grid(nbi * nbj * vtiles * nseg, 1);
  CUtensorMap map;
  cuuint64_t gd[4] = {(cuuint64_t)W, 2, (cuuint64_t)H, 1}, gs[3] = {(cuuint64_t)W * 8, (cuuint64_t)W * 16, (cuuint64_t)H * W * 16};
  cuuint32_t bx[4] = {(cuuint32_t)tc::kBoxW, 2, 1, 1}, es[4] = {1, 1, 1, 1};
  CUresult cr = cuTensorMapEncodeTiled(&map, CU_TENSOR_MAP_DATA_TYPE_UINT64, 4, img, gd, gs, bx, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                                       CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
                                       CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (cr != CUDA_SUCCESS) { printf("encode failed %d\n", (int)cr); return 1; }
  for (int it = 0; it < 3; ++it) tm_tc_kernel<<<grid, tc::kThreads, smem>>>(a, map);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0); cudaEventCreate(&e1);
  cudaEventRecord(e0);
  tm_tc_kernel<<<grid, tc::kThreads, smem>>>(a, map);
  cudaEventRecord(e1);
  cudaError_t e = cudaDeviceSynchronize();
  float ms = 0; cudaEventElapsedTime(&ms, e0, e1);
  std::vector<long long> t(8 * 1024);
  cudaMemcpy(t.data(), tr, t.size() * 8, cudaMemcpyDeviceToHost);
  printf("{\"err\": \"%s\", \"exp\": %d, \"ms\": %.4f, \"grid\": %d}\n", cudaGetErrorString(e), exp, ms, grid.x);
  const long long t0 = t[3 * 1024];
  // per stage q of one producer group: img_full passed, split done, mma_done(q - 6) passed (stamp 0 of
  // q - 6), arrive; the MMA warp's start and commit of q
  for (int q = 100; q < 104; ++q)
    printf("q=%3d  img_full_ok=%8lld  split=%8lld  done(q-6)_ok=%8lld  arrive=%8lld  mma_go=%8lld  commit=%8lld\n", q,
           t[5 * 1024 + q] - t0, t[1024 + q] - t0, t[q - 6] - t0, t[2048 + q] - t0, t[3072 + q] - t0, t[4096 + q] - t0);
  for (int q = 100; q < 104; ++q)
    printf("q=%3d  prod_wait_done(q)=%8lld  prod_split(q)=%8lld  prod_arrive(q)=%8lld  mma_go(q)=%8lld  mma_commit(q)=%8lld\n", q,
           t[q] - t0, t[1024 + q] - t0, t[2048 + q] - t0, t[3072 + q] - t0, t[4096 + q] - t0);
  // MMA warp per row group g: group start (after the previous group's commit), drained wait passed,
  // first and last stage start
  for (int g = 10; g < 16; ++g)
    printf("g=%2d  start=%8lld  drained_ok=%8lld  first_go=%8lld  last_commit=%8lld\n", g, t[6 * 1024 + g] - t0,
           t[7 * 1024 + g] - t0, t[3072 + 8 * g] - t0, t[4096 + 8 * g + 7] - t0);
  // steady-state averages over stages 40..300
  double d_go = 0, d_arr = 0, d_done = 0;
  for (int q = 41; q < 300; ++q) {
    d_go += t[3072 + q] - t[3072 + q - 1];
    d_arr += t[2048 + q] - t[2048 + q - 1];
    d_done += t[q] - t[q - 1];
  }
  printf("avg cycles/stage: mma_go %.1f  prod_arrive %.1f  mma_done %.1f\n", d_go / 259, d_arr / 259, d_done / 259);
  double lag = 0, split = 0, stw = 0;
  for (int q = 41; q < 300; ++q) {
    lag += t[3072 + q] - t[2048 + q];       // arrive -> MMA thread sees it
    split += t[1024 + q] - t[q - 4 >= 0 ? q - 4 : 0];
    stw += t[2048 + q] - t[1024 + q];       // LDG issue + TMEM stores + wait
  }
  printf("avg: arrive->mma_go %.1f  split->arrive %.1f\n", lag / 259, stw / 259);
  // per-region stage times of CTA 0 (mma_go(q+1) - mma_go(q)): ramp-in, middle, ramp-out rows
  {
    const int nu = (U + nseg - 1) / nseg, R = nu + tc::kHB - 1;
    const int nst = ((R + tc::kG - 1) / tc::kG) * tc::kG * (WC / tc::kWB);
    const int per_row = WC / tc::kWB;
    double rin = 0, mid = 0, rout = 0;
    int nin = 0, nmid = 0, nout = 0;
    for (int q = 1; q < nst && q < 1024; ++q) {
      const double d = (double)(t[3072 + q] - t[3072 + q - 1]);
      const int row = q / per_row;
      if (row < tc::kHB - 1) { rin += d; ++nin; }
      else if (row < nu) { mid += d; ++nmid; }
      else { rout += d; ++nout; }
    }
    printf("stages %d: ramp-in %.1f (%d)  middle %.1f (%d)  ramp-out %.1f (%d)  total %lld cycles\n", nst,
           nin ? rin / nin : 0, nin, nmid ? mid / nmid : 0, nmid, nout ? rout / nout : 0, nout,
           (long long)(t[4096 + (nst < 1024 ? nst : 1024) - 1] - t[3072]));
  }
  return 0;
}
