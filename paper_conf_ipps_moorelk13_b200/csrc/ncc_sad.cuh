// ncc_sad.cuh -- sum of absolute differences (SAD) for TM and PIV.
//
// SAD(u, v) = sum_{i<h, j<w} |T[i][j] - I[u+i][v+j]|: the paper's own specialisation example
// swaps exactly this metric for the sum of squared differences (Ch. 4), and both
// are the classic block-matching scores beside correlation (the paper's PIV metric is SSD,
// Fig 5.10 caption P:167-168).  Unlike NCC and SSD it has no numerator / window-sum
// decomposition (|.| is not bilinear), so it cannot use the tensor cores or the FFMA2
// correlation cores: these kernels form every |t - b| directly on the CUDA cores (FADD with the
// |.| operand modifier), fp32 with a fresh partial per template row (the accumulation order of
// the FFMA kernels), peak = argmin with the same packed-key tie rule, PIV sub-pixel = the
// parabola through the minimum (as SSD).
#pragma once
#include "ncc_kernels.cuh"

namespace nccb {

constexpr int kSadTU = 16, kSadTV = 64, kSadRV = 4, kSadCH = 8;  // TM tile: 16 x 64 offsets, 4 per thread

// TM SAD: grid = (ceil(V / 64), ceil(Ub / 16), batch), block = 256 (16 rows x 16 column groups).
// Template rows are staged kSadCH at a time with the image rows they touch; each thread slides
// a 4-value register window along its image row (one shared load per template column).
// dynamic smem = kSadCH * w + (kSadCH + kSadTU - 1) * (kSadTV + w - 1 + 3) floats.
__global__ void __launch_bounds__(256) tm_sad_kernel(const float* __restrict__ img, int64_t pitch,
                                                     int64_t frame_stride, int H, int W,
                                                     const float* __restrict__ tmpl, int64_t tpitch, int h, int w,
                                                     int u_begin, int Ub, int V, float* scores,
                                                     int64_t score_frame_stride, unsigned long long* keys) {
  extern __shared__ float sm_sad[];
  const int IW = kSadTV + w - 1 + 3;  // staged image row (columns v0 .. v0 + 63 + w - 1, padded)
  float* Ts = sm_sad;                 // [kSadCH][w]
  float* Is = sm_sad + kSadCH * w;    // [kSadCH + kSadTU - 1][IW]
  const int f = blockIdx.z;
  const int ur0 = blockIdx.y * kSadTU, v0 = blockIdx.x * kSadTV;
  const int ty = threadIdx.x >> 4, tx = threadIdx.x & 15;
  const float* I = img + (int64_t)f * frame_stride;
  float tot[kSadRV];
#pragma unroll
  for (int r = 0; r < kSadRV; ++r) tot[r] = 0.0f;
  for (int i0 = 0; i0 < h; i0 += kSadCH) {
    const int ch = min(kSadCH, h - i0);
    __syncthreads();
    for (int e = threadIdx.x; e < ch * w; e += 256) Ts[e] = __ldg(tmpl + (int64_t)(i0 + e / w) * tpitch + e % w);
    const int rows = ch + kSadTU - 1;
    for (int e = threadIdx.x; e < rows * IW; e += 256) {
      const int rr = e / IW, cc = e % IW;
      const int gy = u_begin + ur0 + i0 + rr, gx = v0 + cc;
      Is[e] = (gy < H && gx < W) ? __ldg(I + (int64_t)gy * pitch + gx) : 0.0f;
    }
    __syncthreads();
    for (int ci = 0; ci < ch; ++ci) {
      const float* tr = Ts + ci * w;
      const float* ir = Is + (ty + ci) * IW + tx * kSadRV;
      float x0 = ir[0], x1 = ir[1], x2 = ir[2];
      float pr[kSadRV];
#pragma unroll
      for (int r = 0; r < kSadRV; ++r) pr[r] = 0.0f;  // fresh partial per template row
      for (int j = 0; j < w; ++j) {
        const float t = tr[j], x3 = ir[j + 3];
        pr[0] += fabsf(t - x0);
        pr[1] += fabsf(t - x1);
        pr[2] += fabsf(t - x2);
        pr[3] += fabsf(t - x3);
        x0 = x1;
        x1 = x2;
        x2 = x3;
      }
#pragma unroll
      for (int r = 0; r < kSadRV; ++r) tot[r] += pr[r];
    }
  }
  const int ur = ur0 + ty;
  unsigned long long best = 0ull;
  if (ur < Ub) {
#pragma unroll
    for (int r = 0; r < kSadRV; ++r) {
      const int v = v0 + tx * kSadRV + r;
      if (v < V) {
        if (scores) scores[(int64_t)f * score_frame_stride + (int64_t)ur * V + v] = tot[r];
        const unsigned long long k = make_key(-tot[r], (uint32_t)((int64_t)(u_begin + ur) * V + v));
        best = k > best ? k : best;
      }
    }
  }
  best = warp_max_key(best);
  if ((threadIdx.x & 31) == 0 && best && best > __ldcg(keys + f)) atomicMax(keys + f, best);
}

__global__ void tm_keys_reset(unsigned long long* keys, int n) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) keys[i] = 0ull;
}

// PIV SAD: one CTA per (window, pair); the mask (frame A) and its search region (frame B) staged
// in shared memory; each thread takes 4 consecutive dx offsets of one dy (register window as in
// tm_sad_kernel), the SAD surface stays in shared memory for the argmin and the parabolic
// sub-pixel fit of the minimum.  grid = (Ky * Kx, pairs), block = 256; dynamic smem =
// h * w + (h + 2 m_y) * RP + OY * OXP floats, RP = w + 2 m_x + 3 (padded), OXP = 4 ceil(OX / 4).
__global__ void __launch_bounds__(256) piv_sad_kernel(const PivArgs a) {
  extern __shared__ float sm_ps[];
  const int h = a.h, w = a.w, my = a.my, mx = a.mx;
  const int OY = 2 * my + 1, OX = 2 * mx + 1, OXP = ((OX + 3) / 4) * 4, NGX = OXP / 4;
  const int BR = h + 2 * my, RP = w + 2 * mx + 3;
  float* Ts = sm_ps;
  float* Rs = Ts + h * w;
  float* Ss = Rs + BR * RP;
  __shared__ unsigned long long red[32];
  const int lin = blockIdx.x, pz = blockIdx.y;
  const int y = my + (lin / a.Kx) * a.sy, x = mx + (lin % a.Kx) * a.sx;
  const float* A = a.A + (int64_t)pz * a.frame_stride;
  const float* B = a.B + (int64_t)pz * a.frame_stride;
  for (int e = threadIdx.x; e < h * w; e += blockDim.x)
    Ts[e] = __ldg(A + (int64_t)(y + e / w) * a.pitch + x + e % w);
  for (int e = threadIdx.x; e < BR * RP; e += blockDim.x) {
    const int rr = e / RP, cc = e % RP;
    Rs[e] = cc < w + 2 * mx ? __ldg(B + (int64_t)(y - my + rr) * a.pitch + x - mx + cc) : 0.0f;
  }
  __syncthreads();
  unsigned long long best = 0ull;
  for (int it = threadIdx.x; it < OY * NGX; it += blockDim.x) {
    const int oy = it / NGX, ox0 = (it % NGX) * 4;
    float tot[4] = {0.0f, 0.0f, 0.0f, 0.0f};
    for (int i = 0; i < h; ++i) {
      const float* tr = Ts + i * w;
      const float* br = Rs + (oy + i) * RP + ox0;
      float x0 = br[0], x1 = br[1], x2 = br[2];
      float pr[4] = {0.0f, 0.0f, 0.0f, 0.0f};  // fresh partial per template row
      for (int j = 0; j < w; ++j) {
        const float t = tr[j], x3 = br[j + 3];
        pr[0] += fabsf(t - x0);
        pr[1] += fabsf(t - x1);
        pr[2] += fabsf(t - x2);
        pr[3] += fabsf(t - x3);
        x0 = x1;
        x1 = x2;
        x2 = x3;
      }
#pragma unroll
      for (int r = 0; r < 4; ++r) tot[r] += pr[r];
    }
#pragma unroll
    for (int r = 0; r < 4; ++r) {
      const int ox = ox0 + r;
      if (ox < OX) {
        Ss[oy * OXP + ox] = tot[r];
        if (a.scores) a.scores[((int64_t)(a.pair0 + pz) * a.Ky * a.Kx + lin) * OY * OX + oy * OX + ox] = tot[r];
        const unsigned long long k = make_key(-tot[r], (uint32_t)(oy * OX + ox));
        best = k > best ? k : best;
      }
    }
  }
  best = block_max_key(best, red);
  __syncthreads();  // the surface in shared memory is complete
  if (threadIdx.x != 0) return;
  const uint32_t kk = key_index(best);
  const int row = (int)(kk / OX), col = (int)(kk % OX);
  const int iy = row - my, ix = col - mx;
  uint32_t flags = 0u;
  double ddy = 0.0, ddx = 0.0;
  if (row == 0 || row == OY - 1) flags |= kEdgeY;
  else ddy = subpix3_min(Ss[(row - 1) * OXP + col], Ss[row * OXP + col], Ss[(row + 1) * OXP + col], a.subpix);
  if (col == 0 || col == OX - 1) flags |= kEdgeX;
  else ddx = subpix3_min(Ss[row * OXP + col - 1], Ss[row * OXP + col], Ss[row * OXP + col + 1], a.subpix);
  VecOut o;
  o.iy = iy;
  o.ix = ix;
  o.dy = (float)(iy + ddy);
  o.dx = (float)(ix + ddx);
  o.score = -key_score(best);
  o.flags = flags;
  a.vec[(int64_t)(a.pair0 + pz) * a.Ky * a.Kx + lin] = o;
}

}  // namespace nccb
