// ncc_kernels.cuh -- sm_100a kernels of the spatial-domain NCC hot path.
//
// Paper: /root/reference/PAPER.md (N. Moore, kernel specialisation dissertation / IPDPS-W'13).
//   Fig 5.1 caption  P:132-137  corr2 / Pearson, A-bar and B-bar matrix averages.
//   Fig 5.2 caption  P:138-146  staged form: B-bar window mean, A_C = template - mean,
//                               A_D = template's denominator contribution.
//   Fig 5.3 caption  P:147-153  numerator stage  sum A_C * B  (sum A_C = 0).
//   Figs 5.4-5.6     P:154-160  template tiles applied to a shift area; one thread per shift
//                               accumulating all tile contributions (here: RV shifts/thread).
//   Fig 2.2          P:448-519  in-block reduction (here: warp redux + packed argmax key).
//   Ch. 4            P:964-1138 kernel specialisation: problem/implementation parameters as
//                               compile-time constants (here: template args TH/TW/MY/MX, 0 =
//                               run-time evaluated "RE" generic kernel, App. B pattern P:1049-1104).
//
// Design (B200): FP32 numerator on CUDA cores (FFMA), template-row-outer loop so every lane
// of the CTA reads the same template value (smem broadcast), each lane owns RV consecutive
// shifts of one output row and slides a register window along the image row (one LDS.128
// of image + one LDS.128 of template per 4 template columns -> 4*RV FFMA).  Row-blocked
// fp32 partials: each template-row x column-chunk partial starts at 0 and is added to the
// running total, bounding fp32 error growth.  Denominator from fp64 window
// sums; normalisation in fp64; packed 64-bit (score, -index) keys for a deterministic argmax.
#pragma once
#ifdef __CUDACC_RTC__
// Run-time specialisation (NVRTC, csrc/ncc_jit.inc): no host headers; the few types used here.
typedef int int32_t;
typedef unsigned int uint32_t;
typedef long long int64_t;
typedef unsigned long long uint64_t;
struct alignas(64) CUtensorMap_st {
  unsigned long long opaque[16];
};
typedef CUtensorMap_st CUtensorMap;
#else
#include <cuda.h>  // CUtensorMap (type only; encoded on the host through the runtime entry point)
#include <cuda_runtime.h>
#include <stdint.h>
#endif

namespace nccb {

constexpr double kFlatRel = 1e-10;  // SURVEY 8(c) reading 4

// Flag bits: identical values to include/ncc.h (interface constants).
constexpr uint32_t kFlatTemplate = 1u, kEdgeY = 2u, kEdgeX = 4u, kParabolaY = 8u, kParabolaX = 16u,
                   kInvalid = 32u;

struct TemplateStats {
  double sum;     // sum T
  double sumsq;   // sum T^2
  double energy;  // A_D = sum (T - Tbar)^2            (Fig 5.2)
  double csum;    // sum of the fp32-rounded A_C values (~0; corrects sum A_C * B exactly)
  int flat;       // A_D <= 1e-10 * sum T^2
  int pad;
};

struct PeakOut {  // == ncc_peak
  float score;
  int32_t u, v;
  uint32_t flags;
};
struct VecOut {  // == piv_vector
  int32_t iy, ix;
  float dy, dx;
  float score;
  uint32_t flags;
};

// ------------------------------------------------------------------ small helpers
__device__ __forceinline__ double warp_sum_d(double v) {
#pragma unroll
  for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}

// Deterministic block sum (fixed shuffle tree, then warp partials in warp order).
// `red` holds >= 32 doubles of shared memory.  All threads get the result.
__device__ __forceinline__ double block_sum_d(double v, double* red) {
  v = warp_sum_d(v);
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5, nw = (blockDim.x + 31) >> 5;
  __syncthreads();
  if (lane == 0) red[wid] = v;
  __syncthreads();
  double r = 0.0;
  for (int k = 0; k < nw; ++k) r += red[k];
  return r;
}

// Orderable 64-bit key: high word = order-preserving image of the fp32 score, low word =
// 0xFFFFFFFF - linear index, so max(key) = max score, ties -> smallest index.
__device__ __forceinline__ unsigned long long make_key(float s, uint32_t idx) {
  const uint32_t b = __float_as_uint(s);
  const uint32_t o = (b & 0x80000000u) ? ~b : (b | 0x80000000u);
  return ((unsigned long long)o << 32) | (unsigned long long)(0xFFFFFFFFu - idx);
}
__device__ __forceinline__ float key_score(unsigned long long k) {
  const uint32_t o = (uint32_t)(k >> 32);
  const uint32_t b = (o & 0x80000000u) ? (o & 0x7FFFFFFFu) : ~o;
  return __uint_as_float(b);
}
__device__ __forceinline__ uint32_t key_index(unsigned long long k) {
  return 0xFFFFFFFFu - (uint32_t)(k & 0xFFFFFFFFull);
}
__device__ __forceinline__ unsigned long long warp_max_key(unsigned long long k) {
  const uint32_t hi = (uint32_t)(k >> 32), lo = (uint32_t)k;
  const uint32_t mh = __reduce_max_sync(0xffffffffu, hi);
  const uint32_t ml = __reduce_max_sync(0xffffffffu, hi == mh ? lo : 0u);
  return ((unsigned long long)mh << 32) | ml;
}
// Block-wide max key; `red` holds >= 32 u64.  Result valid in thread 0 (and returned to all).
__device__ __forceinline__ unsigned long long block_max_key(unsigned long long k, unsigned long long* red) {
  k = warp_max_key(k);
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5, nw = (blockDim.x + 31) >> 5;
  __syncthreads();
  if (lane == 0) red[wid] = k;
  __syncthreads();
  unsigned long long r = 0;
  for (int q = 0; q < nw; ++q) r = red[q] > r ? red[q] : r;
  return r;
}

// NCC from the numerator and fp64 window sums (Fig 5.1/5.2): the centred numerator is
// sum A_C (B - Bbar) = sum A_C B - (sum A_C) * S1 / n; the fp32 A_C sum is ~1e-6, but
// subtracting it makes the identity exact for the stored A_C.
__device__ __forceinline__ float ncc_normalize(float num, double s1, double s2, double n,
                                               const TemplateStats& ts) {
  const double var = s2 - s1 * s1 / n;  // n * window variance
  if (ts.flat || !(var > kFlatRel * s2)) return 0.0f;
  double r = ((double)num - ts.csum * s1 / n) / sqrt(ts.energy * var);
  r = r > 1.0 ? 1.0 : (r < -1.0 ? -1.0 : r);
  return (float)r;
}


// ------------------------------------------------------------------ TMA / mbarrier (sm_100a PTX)
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred P;\n"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1;\n\t"
      "@!P bra WAIT_%=;\n}" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}
// Bounded wait for the warp-specialised pipelines: a protocol bug traps (launch error)
// instead of hanging the device.
__device__ __forceinline__ void mbar_wait_bounded(uint64_t* bar, uint32_t parity) {
  uint32_t done = 0;
  for (long long it = 0; it < (1ll << 30); ++it) {
    asm volatile(
        "{\n\t.reg .pred P;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 P, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, P;\n}"
        : "=r"(done)
        : "r"(smem_u32(bar)), "r"(parity)
        : "memory");
    if (done) return;
  }
  __trap();
}
// Long waits of otherwise idle warps (a producer waiting for a window's core): back off with
// nanosleep so the spinning does not take issue slots from the warps doing the work.
__device__ __forceinline__ void mbar_wait_backoff(uint64_t* bar, uint32_t parity) {
  uint32_t done = 0, ns = 64;
  for (long long it = 0; it < (1ll << 26); ++it) {
    asm volatile(
        "{\n\t.reg .pred P;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 P, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, P;\n}"
        : "=r"(done)
        : "r"(smem_u32(bar)), "r"(parity)
        : "memory");
    if (done) return;
    __nanosleep(ns);
    ns = ns < 2048 ? 2 * ns : ns;
  }
  __trap();
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void named_bar_sync(int id, int nthreads) {
  asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}
// 2D / 3D tiled TMA loads global -> shared, completion on an mbarrier (out-of-bounds = 0).
__device__ __forceinline__ void tma_load_2d(void* dst, const CUtensorMap* map, int x, int y, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::
          "r"(smem_u32(dst)),
      "l"(map), "r"(x), "r"(y), "r"(smem_u32(bar))
      : "memory");
}
__device__ __forceinline__ void tma_load_3d(void* dst, const CUtensorMap* map, int x, int y, int z, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], [%5];" ::
          "r"(smem_u32(dst)),
      "l"(map), "r"(x), "r"(y), "r"(z), "r"(smem_u32(bar))
      : "memory");
}
__device__ __forceinline__ void tma_load_4d(void* dst, const CUtensorMap* map, int x, int y, int z, int w, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.tensor.4d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5}], [%6];" ::
          "r"(smem_u32(dst)),
      "l"(map), "r"(x), "r"(y), "r"(z), "r"(w), "r"(smem_u32(bar))
      : "memory");
}
__device__ __forceinline__ void tma_prefetch_desc(const CUtensorMap* map) {
  asm volatile("prefetch.tensormap [%0];" ::"l"(map) : "memory");
}

// ------------------------------------------------------------------ numerator core
// acc[c] += sum_{j<CW} tpl[j] * img[c + j],  c < RV.
// img: shared, 16-B aligned, >= RV + CW readable values; tpl: shared, 16-B aligned (broadcast).
// One LDS.128 of image and one of template per 4 columns; the register window slides by
// renaming (full unroll), so the inner body is 4*RV FFMA per 2 LDS.
template <int RV, int CW>
__device__ __forceinline__ void row_dot(const float* __restrict__ img, const float* __restrict__ tpl,
                                        float (&acc)[RV]) {
  static_assert(RV % 4 == 0 && CW % 4 == 0, "RV and CW must be multiples of 4");
  float x[RV];
#pragma unroll
  for (int c = 0; c < RV; c += 4) {
    const float4 v = *reinterpret_cast<const float4*>(img + c);
    x[c] = v.x; x[c + 1] = v.y; x[c + 2] = v.z; x[c + 3] = v.w;
  }
#pragma unroll
  for (int j = 0; j < CW; j += 4) {
    const float4 nx = *reinterpret_cast<const float4*>(img + RV + j);
    const float4 t = *reinterpret_cast<const float4*>(tpl + j);
    const float tt[4] = {t.x, t.y, t.z, t.w};
    const float nn[4] = {nx.x, nx.y, nx.z, nx.w};
#pragma unroll
    for (int s = 0; s < 4; ++s) {
#pragma unroll
      for (int c = 0; c < RV; ++c) acc[c] = fmaf(tt[s], x[c], acc[c]);
#pragma unroll
      for (int c = 0; c < RV - 1; ++c) x[c] = x[c + 1];
      x[RV - 1] = nn[s];
    }
  }
}

// Bank-conflict model for the image LDS.128 of row_dot: a warp's 128-bit loads are served
// in 4 phases of 8 lanes; lane l reads 16 B at float offset (row(l) * pitch + col(l)).
// Returns the worst number of lanes of one phase that hit the same 4-bank group.
__host__ __device__ constexpr int lds128_worst(int RV, int LX, int pitch) {
  int worst = 1;
  for (int p = 0; p < 4; ++p) {
    int cnt[8] = {0, 0, 0, 0, 0, 0, 0, 0};
    for (int l = 8 * p; l < 8 * p + 8; ++l) {
      const int ly = l / LX, lx = l % LX;
      const int g = ((ly * pitch + lx * RV) / 4) % 8;
      cnt[g]++;
      if (cnt[g] > worst) worst = cnt[g];
    }
  }
  return worst;
}
__host__ __device__ constexpr int pick_pitch(int minp, int RV, int LX) {
  const int p0 = (minp + 3) & ~3;
  for (int p = p0; p < p0 + 32; p += 4)
    if (lds128_worst(RV, LX, p) == 1) return p;
  return p0;
}

// ================================================================== TM kernels
struct TmArgs {
  const float* img;          // frames, row pitch `pitch`, frame stride `frame_stride` (elements)
  int64_t pitch, frame_stride;
  int H, W;
  const float* tplC;         // centred template, zero-padded to [nCH*CH][tplP]
  int tplP;
  int h, w, nCH, nCW;        // run-time template dims and chunk counts (RE path)
  const double* S1;          // window sums over the band: [batch][u_end-u_begin][V]
  const double* S2;
  int64_t stat_frame_stride;
  const TemplateStats* tst;
  int U, V, u_begin, u_end;
  int tiles_u, tiles_v;      // output tiles of the band
  float* scores;             // nullable: [batch][u_end-u_begin][V]
  int64_t score_frame_stride;
  unsigned long long* keys;  // [batch] argmax keys (reset by tm_template_prep)
  float* part;               // split-K partial totals [batch][tiles][S][RV][NT]   (S > 1)
  unsigned int* cnt;         // split-K arrival counters [batch][tiles], zero between calls
  int S;                     // split-K factor (fixed per problem: accumulation order depends on it)
  // constant-template slabs: this launch covers chunks [q_begin, q_end) of every tile; the
  // template rows [c_row0, c_row0 + rows) are resident in c_tpl (pitch tplP).  A running
  // total is carried between slab launches in `carry` ([batch][tiles][RV][NT]).
  int q_begin, q_end, c_row0, first, last;
  float* carry;
  int ssd;                   // 0: NCC (argmax), 1: SSD = sum (T - W)^2 (argmin; Fig 5.10)
  // multi-template / ROI mode (TM runtime operation: several templates per frame, each searched
  // inside its region of interest; Tab 5.1, 5.1.3.4 P:91).  blockIdx.y = frame*n_tmpl + t.
  int n_tmpl;                // >= 1
  const int* roi;            // nullable: [batch][n_tmpl][2] offset-space ROI origins (u0, v0)
  int roi_h, roi_w;          // ROI extent in offsets (ROI mode)
  int64_t tpl_stride;        // floats between consecutive centred templates (tplC and c_tpl)
  int tpl_rows;              // padded rows per template (TMA row offset of template t)
  int map_u0;                // first offset row held in S1/S2 (band start; 0 in ROI mode)
};

// Template chunks in the constant bank: FFMA takes the template from uniform registers
// (LDCU), so each FFMA reads only two vector registers and the register-bank conflicts
// of the shared-memory-template form (ncu 'dispatch stall', tools/sass_banks.py) vanish.
constexpr int kConstTplFloats = 16384;  // 64 KB
__constant__ float c_tpl[kConstTplFloats];

template <int RV, int CW>
__device__ __forceinline__ void row_dot_c(const float* __restrict__ img, int toff, float (&acc)[RV]) {
  float x[RV];
#pragma unroll
  for (int c = 0; c < RV; c += 4) {
    const float4 v = *reinterpret_cast<const float4*>(img + c);
    x[c] = v.x; x[c + 1] = v.y; x[c + 2] = v.z; x[c + 3] = v.w;
  }
#pragma unroll
  for (int j = 0; j < CW; j += 4) {
    const float4 nx = *reinterpret_cast<const float4*>(img + RV + j);
    const float tt[4] = {c_tpl[toff + j], c_tpl[toff + j + 1], c_tpl[toff + j + 2], c_tpl[toff + j + 3]};
    const float nn[4] = {nx.x, nx.y, nx.z, nx.w};
#pragma unroll
    for (int s = 0; s < 4; ++s) {
#pragma unroll
      for (int c = 0; c < RV; ++c) acc[c] = fmaf(tt[s], x[c], acc[c]);
#pragma unroll
      for (int c = 0; c < RV - 1; ++c) x[c] = x[c + 1];
      x[RV - 1] = nn[s];
    }
  }
}

template <int RV, int LX, int WX, int WY, int CH, int CW>
struct TmTile {
  static constexpr int NT = WX * WY * 32;
  static constexpr int LY = 32 / LX;
  static constexpr int BU = WY * LY;              // output rows per CTA
  static constexpr int BV = WX * LX * RV;         // output cols per CTA
  static constexpr int IR = BU + CH - 1;          // staged image rows (= TMA box rows)
  static constexpr int IP = pick_pitch(BV + CW, RV, LX);  // staged image pitch (= TMA box cols)
  static constexpr int T_BYTES = CH * CW * 4;
  static constexpr int I_BYTES = IR * IP * 4;
  static constexpr int T_AL = ((T_BYTES + 127) / 128) * 128;
  static constexpr int I_AL = ((I_BYTES + 127) / 128) * 128;
  __host__ __device__ static constexpr int stage(bool ct) { return (ct ? 0 : T_AL) + I_AL; }
  __host__ __device__ static constexpr int smem_tma(bool ct) { return 2 * stage(ct); }  // double-buffered
  __host__ __device__ static constexpr int smem_ldg(bool ct) { return (ct ? 0 : T_BYTES) + I_BYTES; }
  static_assert(IR <= 256 && IP <= 256 && CW <= 256 && CH <= 256, "TMA box dims are limited to 256");
};

// Numerator + fused normalise / clamp / optional surface store / CTA argmax (Fig 5.3-5.6).
// TH, TW: compile-time template size (specialised, "SK") or 0 (run-time evaluated, "RE").
// CT:  template from the constant bank (slabs of <= 64 KB) instead of shared memory.
// S:   split of the tile's (row-chunk, col-chunk) sequence over S CTAs; ranges are fixed per
//      tile and the S partial totals are combined in index order by the last CTA to arrive, so
//      the result is deterministic and independent of scheduling and of the band (shard).
// TMA: stage image (and template) chunks with double-buffered cp.async.bulk.tensor + mbarrier;
//      otherwise (pitch not 16-B aligned) plain coalesced loads, single buffer.
// Per-offset order: partial per (template row, column chunk) added to the total in chunk
// order; slab launches carry the running total, so the order equals the single-launch one.
// One CTA = one (tile, split) unit: blockIdx.x = tile * S + split, blockIdx.y = frame.
template <int RV, int LX, int WX, int WY, int CH, int CW, int TH, int TW, bool TMA, bool CT>
__global__ void __launch_bounds__(WX* WY * 32)
    tm_ncc_kernel(const TmArgs a, const __grid_constant__ CUtensorMap map_img,
                  const __grid_constant__ CUtensorMap map_tpl) {
  using T = TmTile<RV, LX, WX, WY, CH, CW>;
  extern __shared__ __align__(1024) unsigned char smem_raw[];
  __shared__ unsigned long long red_key[32];
  __shared__ __align__(8) uint64_t full_bar[2];
  __shared__ unsigned int last_flag;

  const int h = TH ? TH : a.h;
  const int w = TW ? TW : a.w;
  const int nCW = TW ? (TW + CW - 1) / CW : a.nCW;
  const int tplP = TW ? ((TW + CW - 1) / CW) * CW : a.tplP;

  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const int wx = wid % WX, wy = wid / WX;
  const int ly = lane / LX, lx = lane % LX;
  const int lu = wy * T::LY + ly;         // local output row
  const int lv = (wx * LX + lx) * RV;     // local output col (first of RV)
  const int ft = blockIdx.y;  // frame * n_tmpl + template
  const int f = ft / a.n_tmpl, tpl = ft % a.n_tmpl;
  const int S = a.S;
  const int tile = blockIdx.x / S, split = blockIdx.x % S;
  const int ty = tile / a.tiles_v, tx = tile % a.tiles_v;
  int ru0 = a.u_begin, rv0 = 0, u_lim = a.u_end, v_lim = a.V;
  if (a.roi) {
    ru0 = a.roi[2 * ft];
    rv0 = a.roi[2 * ft + 1];
    u_lim = min(ru0 + a.roi_h, a.U);
    v_lim = min(rv0 + a.roi_w, a.V);
  }
  // tiles start at a multiple of 4 columns: a TMA box must start on a 16-byte boundary of the
  // row (measured on B200: an unaligned inner coordinate raises an illegal instruction); the
  // ROI's first columns below rv0 are computed and masked (host: tiles_v covers roi_w + 3)
  const int v_org = rv0 & ~3;
  const int v_min = rv0 > 0 ? rv0 : 0;
  const int u0 = ru0 + ty * T::BU;
  const int v0 = v_org + tx * T::BV;
  const int nq = a.q_end - a.q_begin;
  const int q0 = a.q_begin + (split * nq) / S;
  // a tile entirely outside its (clipped) ROI computes nothing (a TMA box may not start past
  // the tensor), but still takes part in the split-K combine
  const int q1 = (u0 >= u_lim || v0 >= v_lim) ? q0 : a.q_begin + ((split + 1) * nq) / S;
  const int64_t tile_lin = (int64_t)ft * a.tiles_u * a.tiles_v + tile;

  float total[RV];
  if (a.first) {
#pragma unroll
    for (int c = 0; c < RV; ++c) total[c] = 0.0f;
  } else {  // continue the running total of the previous slab launch (S == 1)
    const float* cp = a.carry + tile_lin * (RV * T::NT);
#pragma unroll
    for (int c = 0; c < RV; ++c) total[c] = __ldcg(cp + c * T::NT + tid);
  }

  auto compute_chunk = [&](int q, const float* Ts, const float* Is) {
    const float* irow = Is + lu * T::IP + lv;
    const int ic = q / nCW, jc = q % nCW;
#pragma unroll 1
    for (int i = 0; i < CH; ++i) {
      float part[RV];
#pragma unroll
      for (int c = 0; c < RV; ++c) part[c] = 0.0f;
      if constexpr (CT)
        row_dot_c<RV, CW>(irow + i * T::IP, (int)(tpl * a.tpl_stride) + (ic * CH + i - a.c_row0) * tplP + jc * CW,
                          part);
      else
        row_dot<RV, CW>(irow + i * T::IP, Ts + i * CW, part);
#pragma unroll
      for (int c = 0; c < RV; ++c) total[c] += part[c];
    }
  };

  if constexpr (TMA) {
    constexpr int STG = T::stage(CT);
    auto stage_t = [&](int s) { return reinterpret_cast<float*>(smem_raw + s * STG); };
    auto stage_i = [&](int s) { return reinterpret_cast<float*>(smem_raw + s * STG + (CT ? 0 : T::T_AL)); };
    auto issue = [&](int q, int s) {  // one thread: chunk q -> stage s
      const int ic = q / nCW, jc = q % nCW;
      mbar_expect_tx(&full_bar[s], (uint32_t)((CT ? 0 : T::T_BYTES) + T::I_BYTES));
      if constexpr (!CT) tma_load_2d(stage_t(s), &map_tpl, jc * CW, tpl * a.tpl_rows + ic * CH, &full_bar[s]);
      tma_load_3d(stage_i(s), &map_img, v0 + jc * CW, u0 + ic * CH, f, &full_bar[s]);
    };
    if (tid == 0) {
      tma_prefetch_desc(&map_img);
      if constexpr (!CT) tma_prefetch_desc(&map_tpl);
      mbar_init(&full_bar[0], 1);
      mbar_init(&full_bar[1], 1);
      fence_mbar_init();
    }
    __syncthreads();
    if (tid == 0) {
      if (q0 < q1) issue(q0, 0);
      if (q0 + 1 < q1) issue(q0 + 1, 1);
    }
    for (int q = q0; q < q1; ++q) {
      const int k = q - q0, s = k & 1;
      mbar_wait(&full_bar[s], (uint32_t)((k >> 1) & 1));
      compute_chunk(q, stage_t(s), stage_i(s));
      __syncthreads();  // every warp is done with stage s
      if (tid == 0 && q + 2 < q1) issue(q + 2, s);
    }
  } else {
    float* Ts = reinterpret_cast<float*>(smem_raw);
    float* Is = Ts + (CT ? 0 : CH * CW);
    const float* img = a.img + (int64_t)f * a.frame_stride;
    for (int q = q0; q < q1; ++q) {
      const int ic = q / nCW, jc = q % nCW;
      __syncthreads();
      if constexpr (!CT) {
        const float* tsrc = a.tplC + tpl * a.tpl_stride + (int64_t)(ic * CH) * tplP + jc * CW;
        for (int k = tid; k < CH * CW; k += T::NT) Ts[k] = tsrc[(k / CW) * tplP + (k % CW)];
      }
      const int gr0 = u0 + ic * CH, gc0 = v0 + jc * CW;
      for (int k = tid; k < T::IR * T::IP; k += T::NT) {
        const int r = k / T::IP, c = k % T::IP;
        const int gr = gr0 + r, gc = gc0 + c;
        Is[k] = (gr >= 0 && gc >= 0 && gr < a.H && gc < a.W) ? __ldg(img + (int64_t)gr * a.pitch + gc) : 0.0f;
      }
      __syncthreads();
      compute_chunk(q, Ts, Is);
    }
  }

  if (!a.last) {  // hand the running total to the next slab launch
    float* cp = a.carry + tile_lin * (RV * T::NT);
#pragma unroll
    for (int c = 0; c < RV; ++c) cp[c * T::NT + tid] = total[c];
    return;
  }

  // ---- split-K combine: partials in fixed split order, by the last unit of the tile
  if (S > 1) {
    float* pbase = a.part + tile_lin * S * (RV * T::NT);
#pragma unroll
    for (int c = 0; c < RV; ++c) pbase[(int64_t)split * RV * T::NT + c * T::NT + tid] = total[c];
    __threadfence();
    __syncthreads();
    unsigned int* cnt = a.cnt + tile_lin;
    if (tid == 0) last_flag = (atomicAdd(cnt, 1u) == (unsigned)(S - 1)) ? 1u : 0u;
    __syncthreads();
    if (!last_flag) return;
    __threadfence();
#pragma unroll
    for (int c = 0; c < RV; ++c) {
      float t = 0.0f;
      for (int sp = 0; sp < S; ++sp)
        t += (sp == split) ? total[c] : __ldcg(pbase + (int64_t)sp * RV * T::NT + c * T::NT + tid);
      total[c] = t;
    }
    if (tid == 0) *cnt = 0u;  // ready for the next call (stream-ordered)
  }

  // ---- fused epilogue: normalise, clamp, optional surface, argmax key
  const TemplateStats ts = a.tst[tpl];
  const double n = (double)h * (double)w;
  const int u = u0 + lu;
  unsigned long long best = 0ull;
  if (u >= 0 && u < u_lim) {
    const int64_t rowoff = (int64_t)f * a.stat_frame_stride + (int64_t)(u - a.map_u0) * a.V;
    float* srow = nullptr;
    if (a.scores)
      srow = a.roi ? a.scores + ((int64_t)ft * a.roi_h + (u - ru0)) * a.roi_w - rv0
                   : a.scores + (int64_t)f * a.score_frame_stride + (int64_t)(u - a.u_begin) * a.V;
#pragma unroll
    for (int c = 0; c < RV; ++c) {
      const int v = v0 + lv + c;
      if (v >= v_min && v < v_lim) {
        const double s1 = a.S1[rowoff + v], s2 = a.S2[rowoff + v];
        float sc;
        if (a.ssd)  // sum T^2 - 2 sum T W + sum W^2, with sum T W = sum A_C W + Tbar S1
          sc = (float)(ts.sumsq - 2.0 * ((double)total[c] + ts.sum / n * s1) + s2);
        else
          sc = ncc_normalize(total[c], s1, s2, n, ts);
        if (srow) srow[v] = sc;
        const unsigned long long k = make_key(a.ssd ? -sc : sc, (uint32_t)((int64_t)u * a.V + v));
        best = k > best ? k : best;
      }
    }
  }
  best = block_max_key(best, red_key);
  if (tid == 0 && best) atomicMax(a.keys + ft, best);
}

// Template prep (Fig 5.2): Tbar, A_C = T - Tbar (fp32, zero-padded), A_D = sum A_C^2 (fp64),
// flat flag; resets the per-frame argmax keys.  One CTA, deterministic reductions.
__global__ void __launch_bounds__(1024) tm_template_prep(const float* __restrict__ tmpl, int64_t tpitch, int h, int w,
                                 float* __restrict__ tplC, int HP, int WP, TemplateStats* ts,
                                 unsigned long long* keys, int batch) {
  // blockIdx.x = template index (multi-template mode): template t at tmpl + t*h*tpitch
  const int t = blockIdx.x, T = gridDim.x;
  tmpl += (int64_t)t * h * tpitch;
  tplC += (int64_t)t * HP * WP;
  ts += t;
  __shared__ double red[32];
  const int n = h * w;
  if ((w & 3) == 0 && (WP & 3) == 0 && (tpitch & 3) == 0 && (reinterpret_cast<unsigned long long>(tmpl) & 15) == 0 &&
      (reinterpret_cast<unsigned long long>(tplC) & 15) == 0 && (int)blockDim.x % (w / 4) == 0) {
    // float4 path: thread -> (row slot, 4-column group); rows strided by blockDim / (w / 4)
    const int g4 = w / 4, rs = (int)blockDim.x / g4;
    const int jr = (int)threadIdx.x / g4, jc = ((int)threadIdx.x % g4) * 4;
    double s = 0.0, s2 = 0.0;
#pragma unroll 4
    for (int i = jr; i < h; i += rs) {
      const float4 x = __ldg(reinterpret_cast<const float4*>(tmpl + (int64_t)i * tpitch + jc));
      s += ((double)x.x + (double)x.y) + ((double)x.z + (double)x.w);
      s2 += ((double)x.x * x.x + (double)x.y * x.y) + ((double)x.z * x.z + (double)x.w * x.w);
    }
    s = block_sum_d(s, red);
    s2 = block_sum_d(s2, red);
    const double mean = s / (double)n;
    double e = 0.0, cs = 0.0;
#pragma unroll 4
    for (int i = jr; i < h; i += rs) {
      const float4 x = __ldg(reinterpret_cast<const float4*>(tmpl + (int64_t)i * tpitch + jc));
      const double a0 = (double)x.x - mean, a1 = (double)x.y - mean, a2 = (double)x.z - mean,
                   a3 = (double)x.w - mean;
      e += (a0 * a0 + a1 * a1) + (a2 * a2 + a3 * a3);
      const float4 ac = make_float4((float)a0, (float)a1, (float)a2, (float)a3);
      cs += ((double)ac.x + (double)ac.y) + ((double)ac.z + (double)ac.w);
      *reinterpret_cast<float4*>(tplC + (int64_t)i * WP + jc) = ac;
    }
    // zero padding (columns w .. WP, rows h .. HP)
    for (int k = threadIdx.x; k < HP * WP; k += blockDim.x) {
      const int i = k / WP, j = k % WP;
      if (i >= h || j >= w) tplC[k] = 0.0f;
    }
    e = block_sum_d(e, red);
    cs = block_sum_d(cs, red);
    if (threadIdx.x == 0) {
      ts->sum = s;
      ts->sumsq = s2;
      ts->energy = e;
      ts->csum = cs;
      ts->flat = (e <= kFlatRel * s2) ? 1 : 0;
      ts->pad = 0;
    }
    for (int f = threadIdx.x; f < batch; f += blockDim.x) keys[(int64_t)f * T + t] = 0ull;
    return;
  }
  // loads in batches of 8 per thread (the single CTA is load-latency bound)
  constexpr int LB = 8;
  double s = 0.0, s2 = 0.0;
  for (int k0 = threadIdx.x; k0 < n; k0 += LB * blockDim.x) {
    float x[LB];
#pragma unroll
    for (int r = 0; r < LB; ++r) {
      const int k = k0 + r * blockDim.x;
      x[r] = k < n ? __ldg(tmpl + (int64_t)(k / w) * tpitch + (k % w)) : 0.0f;
    }
#pragma unroll
    for (int r = 0; r < LB; ++r) {
      s += (double)x[r];
      s2 += (double)x[r] * (double)x[r];
    }
  }
  s = block_sum_d(s, red);
  s2 = block_sum_d(s2, red);
  const double mean = s / (double)n;
  double e = 0.0, cs = 0.0;
  for (int k0 = threadIdx.x; k0 < HP * WP; k0 += LB * blockDim.x) {
    float x[LB];
#pragma unroll
    for (int r = 0; r < LB; ++r) {
      const int k = k0 + r * blockDim.x, i = k / WP, j = k % WP;
      x[r] = (k < HP * WP && i < h && j < w) ? __ldg(tmpl + (int64_t)i * tpitch + j) : 0.0f;
    }
#pragma unroll
    for (int r = 0; r < LB; ++r) {
      const int k = k0 + r * blockDim.x, i = k / WP, j = k % WP;
      if (k >= HP * WP) break;
      float ac = 0.0f;
      if (i < h && j < w) {
        const double a = (double)x[r] - mean;
        e += a * a;
        ac = (float)a;
        cs += (double)ac;
      }
      tplC[k] = ac;
    }
  }
  e = block_sum_d(e, red);
  cs = block_sum_d(cs, red);
  if (threadIdx.x == 0) {
    ts->sum = s;
    ts->sumsq = s2;
    ts->energy = e;
    ts->csum = cs;
    ts->flat = (e <= kFlatRel * s2) ? 1 : 0;
    ts->pad = 0;
  }
  for (int f = threadIdx.x; f < batch; f += blockDim.x) keys[(int64_t)f * T + t] = 0ull;
}

__global__ void tm_finalize(const unsigned long long* __restrict__ keys, const TemplateStats* ts, int V,
                            PeakOut* __restrict__ peaks, int batch, int ssd, int n_tmpl) {
  const int f = blockIdx.x * blockDim.x + threadIdx.x;  // frame * n_tmpl + template
  if (f >= batch * n_tmpl) return;
  ts += f % n_tmpl;
  const unsigned long long k = keys[f];
  const uint32_t idx = key_index(k);
  PeakOut p;
  p.score = ssd ? -key_score(k) : key_score(k);
  p.u = (int32_t)(idx / (uint32_t)V);
  p.v = (int32_t)(idx % (uint32_t)V);
  p.flags = (ts->flat && !ssd) ? (kFlatTemplate | kInvalid) : 0u;
  peaks[f] = p;
}

// ================================================================== window sums (a2)
// Per-offset normalisation factors of a window for the tensor-core epilogue (which then needs
// only fp32 arithmetic per output): rsqrt of n x the window variance, S2 - S1^2/n, computed in
// fp64 and rounded once to fp32 (0 for a flat window: var <= 1e-10 S2, as ncc_normalize), and the
// window mean S1/n for the sum(A_C) correction.
__device__ __forceinline__ void window_denoms(double s1, double s2, double inv_n, float* rsv, float* mean) {
  const double var = s2 - s1 * s1 * inv_n;
  *rsv = (var > kFlatRel * s2) ? (float)rsqrt(var) : 0.0f;  // fp64 rsqrt (1 ulp) rounded once to fp32
  *mean = (float)(s1 * inv_n);
}

// Inclusive warp scan (fp64, shuffle-up tree).
__device__ __forceinline__ double warp_incl_scan_d(double v) {
  const int lane = threadIdx.x & 31;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const double t = __shfl_up_sync(0xffffffffu, v, o);
    if (lane >= o) v += t;
  }
  return v;
}

// Horizontal pass: RS[f][r][v] = sum_{j<w} I[row0 + r][v + j] for v < V (fp64), via a
// segment-local fp64 prefix sum staged in shared memory (exact for 2^-8-quantised inputs).
// grid = (ceil(V / seg), rows, batch), block = NT, dynamic smem = 2 * (seg + w + 1) doubles.
template <int NT>
__global__ void __launch_bounds__(NT)
    box_rows_kernel(const float* __restrict__ img, int64_t pitch, int64_t frame_stride, int W, int row0, int w,
                    int V, int seg, double* __restrict__ RS1, double* __restrict__ RS2, int64_t rs_frame_stride) {
  extern __shared__ double sm_d[];
  __shared__ double wt1[NT / 32], wt2[NT / 32];
  const int L = seg + w;  // prefix entries P[0..L-1], P[k] = sum of the first k inputs
  double* P1 = sm_d;
  double* P2 = sm_d + L + 1;
  const int f = blockIdx.z, r = blockIdx.y;
  const int c0 = blockIdx.x * seg;
  const float* src = img + (int64_t)f * frame_stride + (int64_t)(row0 + r) * pitch + c0;
  const int cnt = min(L - 1, W - c0);  // inputs available in this segment
  const int per = (L - 1 + NT - 1) / NT;
  const int b0 = threadIdx.x * per;
  double a1 = 0.0, a2 = 0.0;
  for (int k = 0; k < per; ++k) {
    const int idx = b0 + k;
    if (idx < cnt) {
      const double x = src[idx];
      a1 += x;
      a2 += x * x;
    }
  }
  // block exclusive scan of the per-thread totals: warp shuffle scan + warp totals
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const double i1 = warp_incl_scan_d(a1), i2 = warp_incl_scan_d(a2);
  if (lane == 31) { wt1[wid] = i1; wt2[wid] = i2; }
  __syncthreads();
  double o1 = 0.0, o2 = 0.0;
  for (int q = 0; q < wid; ++q) { o1 += wt1[q]; o2 += wt2[q]; }
  double s1 = o1 + i1 - a1, s2 = o2 + i2 - a2;
  if (threadIdx.x == 0) { P1[0] = 0.0; P2[0] = 0.0; }
  for (int k = 0; k < per; ++k) {
    const int idx = b0 + k;
    if (idx < L - 1) {
      const double x = idx < cnt ? (double)src[idx] : 0.0;
      s1 += x;
      s2 += x * x;
      P1[idx + 1] = s1;
      P2[idx + 1] = s2;
    }
  }
  __syncthreads();
  double* q1 = RS1 + (int64_t)f * rs_frame_stride + (int64_t)r * V;
  double* q2 = RS2 + (int64_t)f * rs_frame_stride + (int64_t)r * V;
  for (int k = threadIdx.x; k < seg; k += NT) {
    const int v = c0 + k;
    if (v < V) {
      q1[v] = P1[k + w] - P1[k];
      q2[v] = P2[k + w] - P2[k];
    }
  }
}

// Fused window sums (one pass, no row-sum intermediate):
//   S[f][u][v] = sum_{i<h, j<w} I[f][row0 + u + i][v + j]  (and of squares), fp64.
// CTA = a strip of TV output columns x TU output rows, processed in sub-blocks of R rows:
//   (1) vertical: each thread owns input columns c of the strip (TV + w - 1 of them) and keeps
//       the column sum CS_u(c) = sum_{i<h} I[u + i][c] in shared memory; the CTA's first row is
//       summed directly (h loads), every later row slides: CS += I[u + h - 1] - I[u - 1];
//   (2) horizontal: one warp per row turns CS into an inclusive prefix P (warp scans with a
//       carry) and writes S[u][v] = P[v + w - 1] - P[v - 1].
// Every partial sum is exact for 2^-8-quantised inputs (any order), so S is exact there.
// grid = (ceil(V / TV), ceil(rows_out / TU), batch), block = NT,
// dynamic smem = (2 * R + 2) * IWP doubles (X1, X2 [R][IWP]; C1, C2 [IWP]).
template <int NT>
__global__ void __launch_bounds__(NT, 2)
    box2d_kernel(const float* __restrict__ img, int64_t pitch, int64_t frame_stride, int row0, int h, int w, int V,
                 int rows_out, int TV, int TU, int R, int IWP, double* __restrict__ S1, double* __restrict__ S2,
                 int64_t s_frame_stride, float* __restrict__ RSV, float* __restrict__ MEAN, double inv_n) {
  extern __shared__ double sm_box[];
  double* X1 = sm_box;
  double* X2 = X1 + (int64_t)R * IWP;
  double* C1 = X2 + (int64_t)R * IWP;
  double* C2 = C1 + IWP;
  const int f = blockIdx.z;
  const int v0 = blockIdx.x * TV;
  const int ub = blockIdx.y * TU;
  const int tv = min(TV, V - v0);
  const int iw = tv + w - 1;
  const int nrow = min(TU, rows_out - ub);
  const float* src = img + (int64_t)f * frame_stride + (int64_t)(row0 + ub) * pitch + v0;
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  constexpr int NW = NT / 32;
  // row layout for the blocked scan: lane k owns the L consecutive columns [k L, k L + L), stored
  // with one pad double per chunk (index c + c / L) so the 32 lanes hit distinct bank pairs
  int lsh = 0;
  while ((32 << lsh) < iw) ++lsh;
  const int L = 1 << lsh;
  auto pidx = [&](int c) { return c + (c >> lsh); };
  // in-frame element offsets and shared-memory indices in 32 bits (a frame's rows x pitch and the
  // staged strip are far below 2^31): one IMAD per load / store instead of 64-bit products
  const int P = (int)pitch, iwp = IWP;
  for (int r0 = 0; r0 < nrow; r0 += R) {
    const int nr = min(R, nrow - r0);
    for (int c = threadIdx.x; c < iw; c += NT) {
      const float* col = src + c;
      double* x1c = X1 + pidx(c);
      double* x2c = X2 + pidx(c);
      double c1, c2;
      int r = 0;
      if (r0 == 0) {  // first output row of the CTA: direct column sum (independent loads)
        double a[4] = {0.0, 0.0, 0.0, 0.0}, b[4] = {0.0, 0.0, 0.0, 0.0};
        int i = 0;
        for (; i + 64 <= h; i += 64) {  // 64 loads in flight, then 4 accumulator chains
          const float* ci = col + i * P;
          float xs[64];
#pragma unroll
          for (int k = 0; k < 64; ++k) xs[k] = __ldg(ci + k * P);
#pragma unroll
          for (int k = 0; k < 64; ++k) {
            const double x = xs[k];
            a[k & 3] += x;
            b[k & 3] = fma(x, x, b[k & 3]);
          }
        }
        for (; i + 32 <= h; i += 32) {  // 32 loads in flight
          const float* ci = col + i * P;
          float xs[32];
#pragma unroll
          for (int k = 0; k < 32; ++k) xs[k] = __ldg(ci + k * P);
#pragma unroll
          for (int k = 0; k < 32; ++k) {
            const double x = xs[k];
            a[k & 3] += x;
            b[k & 3] = fma(x, x, b[k & 3]);
          }
        }
#pragma unroll 8
        for (; i < h; ++i) {
          const double x = __ldg(col + i * P);
          a[0] += x;
          b[0] = fma(x, x, b[0]);
        }
        c1 = (a[0] + a[1]) + (a[2] + a[3]);
        c2 = (b[0] + b[1]) + (b[2] + b[3]);
        x1c[0] = c1;
        x2c[0] = c2;
        r = 1;
      } else {
        c1 = C1[c];
        c2 = C2[c];
      }
      // slide down one row at a time (+ entering row, - leaving row); the loads of up to 16
      // rows are issued before the dependent sums (the sums are a serial chain per column)
      for (; r < nr; r += 16) {
        const float* pin = col + (r0 + r + h - 1) * P;   // entering row of output row r0 + r
        const float* pout = col + (r0 + r - 1) * P;      // leaving row
        float xin[16], xout[16];
#pragma unroll
        for (int k = 0; k < 16; ++k) {
          const bool ok = r + k < nr;
          xin[k] = ok ? __ldg(pin + k * P) : 0.0f;
          xout[k] = ok ? __ldg(pout + k * P) : 0.0f;
        }
        double* s1p = x1c + r * iwp;
        double* s2p = x2c + r * iwp;
#pragma unroll
        for (int k = 0; k < 16; ++k) {
          if (r + k >= nr) break;
          const double xi = xin[k], xo = xout[k];
          c1 = (c1 + xi) - xo;
          c2 = fma(-xo, xo, fma(xi, xi, c2));
          s1p[k * iwp] = c1;
          s2p[k * iwp] = c2;
        }
      }
      C1[c] = c1;
      C2[c] = c2;
    }
    __syncthreads();
    for (int r = wid; r < nr; r += NW) {
      double* x1 = X1 + r * iwp;
      double* x2 = X2 + r * iwp;
      // blocked inclusive prefix: chunk totals, warp scan of the totals, chunk prefixes; the
      // lane's chunk [lane L, lane L + L) is contiguous in the padded row, at lane (L + 1)
      const int cb = lane * L, n = max(0, min(L, iw - cb));
      double* y1 = x1 + lane * (L + 1);
      double* y2 = x2 + lane * (L + 1);
      double t1 = 0.0, t2 = 0.0;
      for (int k = 0; k < n; ++k) {
        t1 += y1[k];
        t2 += y2[k];
      }
      double p1 = warp_incl_scan_d(t1) - t1, p2 = warp_incl_scan_d(t2) - t2;
      for (int k = 0; k < n; ++k) {
        p1 += y1[k];
        p2 += y2[k];
        y1[k] = p1;
        y2[k] = p2;
      }
      __syncwarp();
      // S1 == nullptr: only the fp32 normalisation factors are wanted (tensor-core NCC paths)
      const int64_t oo = (int64_t)f * s_frame_stride + (int64_t)(ub + r0 + r) * V + v0;
      for (int v = lane; v < tv; v += 32) {
        const double s1 = x1[pidx(v + w - 1)] - (v > 0 ? x1[pidx(v - 1)] : 0.0);
        const double s2 = x2[pidx(v + w - 1)] - (v > 0 ? x2[pidx(v - 1)] : 0.0);
        if (S1) {
          S1[oo + v] = s1;
          S2[oo + v] = s2;
        }
        if (RSV) window_denoms(s1, s2, inv_n, RSV + oo + v, MEAN + oo + v);
      }
    }
    __syncthreads();
  }
}

// Vertical pass: S[f][u][v] = sum_{i<h} RS[f][u + i][v] for u < rows_out (fp64).
// CTA = 32 columns (lanes) x NW warps, output rows [ub, ub + NW*L).  The first row's sum is
// formed cooperatively (each warp sums h/NW rows, combined in warp order); the others follow
// from a block scan of the differences d_k = RS[ub+k+h] - RS[ub+k] (warp-local sequential
// scan + exclusive scan of the warp totals).  ~3 loads per output, all warps issue
// independent loads (the sliding form needed h + 2L dependent-latency loads per thread).
// Exact for 2^-8-quantised inputs.  grid = (ceil(V/32), ceil(rows_out/(NW*L)), batch).
template <int NW, int L>
__global__ void __launch_bounds__(NW * 32)
    box_cols_kernel(const double* __restrict__ RS1, const double* __restrict__ RS2, int64_t rs_frame_stride,
                    int V, int h, int rows_out, double* __restrict__ S1, double* __restrict__ S2,
                    int64_t s_frame_stride, float* __restrict__ RSV, float* __restrict__ MEAN, double inv_n) {
  __shared__ double part1[NW][32], part2[NW][32], tot1[NW][32], tot2[NW][32];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const int v = blockIdx.x * 32 + lane;
  const bool okv = v < V;
  const int vv = okv ? v : V - 1;
  const int f = blockIdx.z;
  const int ub = blockIdx.y * (NW * L);
  const double* r1 = RS1 + (int64_t)f * rs_frame_stride + vv;
  const double* r2 = RS2 + (int64_t)f * rs_frame_stride + vv;
  // (1) first output row of the CTA: sum over rows ub .. ub+h-1, split over the warps
  double a1 = 0.0, a2 = 0.0;
  for (int i = wid; i < h; i += NW) {
    a1 += __ldg(r1 + (int64_t)(ub + i) * V);
    a2 += __ldg(r2 + (int64_t)(ub + i) * V);
  }
  part1[wid][lane] = a1;
  part2[wid][lane] = a2;
  // (2) this warp's differences and their local inclusive scan
  const int k0 = wid * L;
  double d1[L], d2[L];
#pragma unroll
  for (int k = 0; k < L; ++k) {
    const int u = ub + k0 + k;  // output row whose difference to the next is d_k
    const bool ok = (u + 1 < rows_out);
    d1[k] = ok ? __ldg(r1 + (int64_t)(u + h) * V) - __ldg(r1 + (int64_t)u * V) : 0.0;
    d2[k] = ok ? __ldg(r2 + (int64_t)(u + h) * V) - __ldg(r2 + (int64_t)u * V) : 0.0;
  }
  double c1 = 0.0, c2 = 0.0;
#pragma unroll
  for (int k = 0; k < L; ++k) {
    c1 += d1[k];
    c2 += d2[k];
    d1[k] = c1;
    d2[k] = c2;
  }
  tot1[wid][lane] = c1;
  tot2[wid][lane] = c2;
  __syncthreads();
  double b1 = 0.0, b2 = 0.0;
  for (int q = 0; q < NW; ++q) {
    b1 += part1[q][lane];
    b2 += part2[q][lane];
  }
  for (int q = 0; q < wid; ++q) {
    b1 += tot1[q][lane];
    b2 += tot2[q][lane];
  }
  // (3) outputs: row ub+k0 gets the base; row ub+k0+k+1 gets base + prefix d_0..d_k
  if (!okv) return;
  double* o1 = S1 + (int64_t)f * s_frame_stride + v;
  double* o2 = S2 + (int64_t)f * s_frame_stride + v;
  if (ub + k0 < rows_out) {
    o1[(int64_t)(ub + k0) * V] = b1;
    o2[(int64_t)(ub + k0) * V] = b2;
    if (RSV) window_denoms(b1, b2, inv_n, RSV + (o1 - S1) + (int64_t)(ub + k0) * V, MEAN + (o1 - S1) + (int64_t)(ub + k0) * V);
  }
#pragma unroll
  for (int k = 0; k + 1 < L; ++k) {
    const int u = ub + k0 + k + 1;
    if (u < rows_out) {
      o1[(int64_t)u * V] = b1 + d1[k];
      o2[(int64_t)u * V] = b2 + d2[k];
      if (RSV) window_denoms(b1 + d1[k], b2 + d2[k], inv_n, RSV + (o1 - S1) + (int64_t)u * V, MEAN + (o1 - S1) + (int64_t)u * V);
    }
  }
}

// ================================================================== PIV kernel (a6, a7)
struct PivArgs {
  const float* A;  // all frames A of the call, row pitch, frame stride in elements
  const float* B;  // all frames B of the call
  int64_t pitch, frame_stride;
  int H, W, h, w, my, mx, sy, sx, Ky, Kx;
  int pair0;         // first pair of this launch (sub-batch); blockIdx.z = pair - pair0
  const double* S1;  // window sums of frame B at every valid position: [pair-pair0][H-h+1][W-w+1]
  const double* S2;
  int64_t map_pitch, map_frame_stride;
  VecOut* vec;       // [pair][Ky][Kx]
  float* scores;     // nullable: [pair][Ky][Kx][OY][OX]
  int subpix;        // 0 Gauss3 (parabolic fallback), 1 parabola, 2 none
  int BP;            // RE: staged B pitch (floats), chosen on the host
  int ssd;           // 0: NCC (argmax), 1: SSD (argmin, parabolic fit of the minimum)
  const float* rsv;  // NCC (nullable): fp32 rsqrt(n var) of frame B's windows (0: flat), S1/map layout
  const float* mean; // ... and the window means S1/n
};

// FFMA2 numerator core with template PAIRS (sm_100a fma.rn.f32x2):
//   acc pair q = (acc[2q+1], acc[2q]);   TP[p] = (t[p-1], t[p]) for p = 0..CW (t[-1] = t[CW] = 0)
//   for every pair p and q:  acc pair q += x[p + 2q] * TP[p]            (x broadcast to both lanes)
// so acc[2q+1] += t[p-1] x[2q+1 + (p-1)] and acc[2q] += t[p] x[2q + p]: exactly sum_j t[j] x[c+j]
// in increasing j (the two boundary products are +0 * x).  Each FFMA2 reads a scalar, a
// template pair and an accumulator pair: with the template pair in the reuse cache it costs
// two register-bank cycles for two FMAs, so bank conflicts cannot throttle the FMA pipe
// (tools/sass_banks.py: 0.85-0.87 vs 0.62 for the scalar shared-memory form).
typedef unsigned long long u64;
__device__ __forceinline__ void ffma2_bcast(u64& d, float x, u64 tp) {
  u64 xx;
  asm("mov.b64 %0, {%1,%1};" : "=l"(xx) : "f"(x));
  asm("fma.rn.f32x2 %0, %1, %2, %0;" : "+l"(d) : "l"(xx), "l"(tp));
}
__device__ __forceinline__ void add2(u64& d, u64 s) { asm("add.rn.f32x2 %0, %0, %1;" : "+l"(d) : "l"(s)); }

template <int RV, int CW>
__device__ __forceinline__ void row_dot_pairs(const float* __restrict__ img, const u64* __restrict__ TP,
                                              u64 (&A2)[RV / 2]) {
  static_assert(RV % 4 == 0 && CW % 4 == 0, "RV and CW must be multiples of 4");
  float x[RV + CW];
#pragma unroll
  for (int c = 0; c < RV; c += 4) {
    const float4 v = *reinterpret_cast<const float4*>(img + c);
    x[c] = v.x; x[c + 1] = v.y; x[c + 2] = v.z; x[c + 3] = v.w;
  }
#pragma unroll
  for (int pp = 0; pp <= CW; pp += 2) {
    if ((pp % 4) == 0 && pp + 4 <= CW) {
      const float4 v = *reinterpret_cast<const float4*>(img + RV + pp);
      x[RV + pp] = v.x; x[RV + pp + 1] = v.y; x[RV + pp + 2] = v.z; x[RV + pp + 3] = v.w;
    }
    const ulonglong2 tp = *reinterpret_cast<const ulonglong2*>(TP + pp);
    const u64 tpv[2] = {tp.x, tp.y};
#pragma unroll
    for (int e = 0; e < 2; ++e) {
      const int p = pp + e;
      if (p <= CW) {
#pragma unroll
        for (int q = 0; q < RV / 2; ++q) ffma2_bcast(A2[q], x[p + 2 * q], tpv[e]);
      }
    }
  }
}

// Same sums, image-major order: for each image value x[c], every (p, q) with p + 2q = c, so
// consecutive FFMA2 share the scalar operand (reuse cache) and read only the template pair and
// the accumulator pair.  Per accumulator the products still come in increasing p.
template <int RV, int CW>
__device__ __forceinline__ void row_dot_pairs_x(const float* __restrict__ img, const u64* __restrict__ TP,
                                                u64 (&A2)[RV / 2]) {
  static_assert(RV % 4 == 0 && CW % 4 == 0, "RV and CW must be multiples of 4");
  float x[RV + CW + 4];
  u64 tp[CW + 2];
#pragma unroll
  for (int c = 0; c < RV + CW; c += 4) {
    const float4 v = *reinterpret_cast<const float4*>(img + c);
    x[c] = v.x; x[c + 1] = v.y; x[c + 2] = v.z; x[c + 3] = v.w;
  }
#pragma unroll
  for (int pp = 0; pp <= CW; pp += 2) {
    const ulonglong2 t = *reinterpret_cast<const ulonglong2*>(TP + pp);
    tp[pp] = t.x;
    tp[pp + 1] = t.y;
  }
#pragma unroll
  for (int c = 0; c < RV + CW; ++c)
#pragma unroll
    for (int q = RV / 2 - 1; q >= 0; --q) {
      const int p = c - 2 * q;
      if (p >= 0 && p <= CW) ffma2_bcast(A2[q], x[c], tp[p]);
    }
}

// Per-window shared-memory geometry (floats); regions rounded to 128 B for TMA destinations.
// TP: template pairs, per row nCW blocks of PB = CW + 2 pairs.  Sc (score tile) aliases TP
// when ALIAS (scores are held in registers across the barrier that ends the numerator).
template <int RV, int CW>
struct PivShape {
  int h, w, my, mx, OY, OX, NG, OXP, nCW, PB, TPP, BR, BP, items, tp_fl, b_fl, s_fl, win_fl;
  __host__ __device__ PivShape(int h_, int w_, int my_, int mx_, int BP_, bool alias)
      : h(h_), w(w_), my(my_), mx(mx_), OY(2 * my_ + 1), OX(2 * mx_ + 1), NG((2 * mx_ + 1 + RV - 1) / RV),
        OXP(((2 * mx_ + 1 + RV - 1) / RV) * RV), nCW((w_ + CW - 1) / CW), PB(CW + 2),
        TPP(((w_ + CW - 1) / CW) * (CW + 2)), BR(h_ + 2 * my_), BP(BP_),
        items((2 * my_ + 1) * ((2 * mx_ + 1 + RV - 1) / RV)) {
    tp_fl = ((h * TPP * 2 + 31) / 32) * 32;
    b_fl = ((BR * BP + 31) / 32) * 32;
    s_fl = ((OY * OXP + 31) / 32) * 32;
    win_fl = (alias ? (tp_fl > s_fl ? tp_fl : s_fl) : tp_fl + s_fl) + b_fl;
  }
  __host__ __device__ int tp_off() const { return 0; }
  __host__ __device__ int b_off(bool alias) const { return alias ? (tp_fl > s_fl ? tp_fl : s_fl) : tp_fl + s_fl; }
  __host__ __device__ int s_off(bool alias) const { return alias ? 0 : tp_fl; }
};

// Bank-conflict model of the PIV image loads (flattened items: lane l -> row l/NG, group l%NG).
__host__ __device__ constexpr int piv_lds128_worst(int RV, int NG, int pitch) {
  int worst = 1;
  for (int p = 0; p < 4; ++p) {
    int cnt[8] = {0, 0, 0, 0, 0, 0, 0, 0};
    for (int l = 8 * p; l < 8 * p + 8; ++l) {
      const int g = (((l / NG) * pitch + (l % NG) * RV) / 4) % 8;
      cnt[g]++;
      if (cnt[g] > worst) worst = cnt[g];
    }
  }
  return worst;
}
__host__ __device__ constexpr int piv_pick_pitch(int minp, int RV, int NG) {
  const int p0 = (minp + 3) & ~3;
  int best = p0, bw = 99;
  for (int p = p0; p < p0 + 32; p += 4) {
    const int wv = piv_lds128_worst(RV, NG, p);
    if (wv < bw) { bw = wv; best = p; }
  }
  return best;
}
__host__ __device__ constexpr int piv_sk_pitch(int TW, int MX, int RV, int CW) {
  return piv_pick_pitch((((2 * MX + 1 + RV - 1) / RV) * RV) + (((TW + CW - 1) / CW) * CW), RV,
                        (2 * MX + 1 + RV - 1) / RV);
}

// Three-point sub-pixel fit along one axis (S8c step 3); fp64 from the fp32 score tile.
__device__ __forceinline__ double subpix3(double cm, double c0, double cp, int mode, bool* parabola) {
  double num, den;
  *parabola = false;
  if (mode == 2) return 0.0;
  if (mode == 0 && cm > 0.0 && c0 > 0.0 && cp > 0.0) {
    const double lm = log(cm), l0 = log(c0), lp = log(cp);
    num = lm - lp;
    den = 2.0 * (lm - 2.0 * l0 + lp);
  } else {
    num = cm - cp;
    den = 2.0 * (cm - 2.0 * c0 + cp);
    *parabola = (mode == 0);
  }
  if (den >= 0.0) return 0.0;
  return num / den;
}
// SSD: three-point parabola through a minimum (0 if not a minimum or mode == none).
__device__ __forceinline__ double subpix3_min(double cm, double c0, double cp, int mode) {
  if (mode == 2) return 0.0;
  const double den = 2.0 * (cm - 2.0 * c0 + cp);
  if (den <= 0.0) return 0.0;
  return (cm - cp) / den;
}

// NCC with the fp64 window sums and a fp32 rsqrt (PIV epilogue): |error| <= ~4e-7 absolute.
__device__ __forceinline__ float ncc_normalize_fast(float num, double s1, double s2, double inv_n, double csum,
                                                    double energy, bool flat) {
  const double var = s2 - s1 * s1 * inv_n;
  if (flat || !(var > kFlatRel * s2)) return 0.0f;
  const float numc = (float)((double)num - csum * s1 * inv_n);
  float r = numc * rsqrtf((float)(energy * var));
  return r > 1.0f ? 1.0f : (r < -1.0f ? -1.0f : r);
}

// Deterministic block sums of K values per thread (red: >= nwarps*K doubles).
template <int K>
__device__ __forceinline__ void block_sum_k(double (&v)[K], double* red) {
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5, nw = (blockDim.x + 31) >> 5;
#pragma unroll
  for (int k = 0; k < K; ++k) v[k] = warp_sum_d(v[k]);
  __syncthreads();
  if (lane == 0) {
#pragma unroll
    for (int k = 0; k < K; ++k) red[wid * K + k] = v[k];
  }
  __syncthreads();
#pragma unroll
  for (int k = 0; k < K; ++k) {
    double r = 0.0;
    for (int q = 0; q < nw; ++q) r += red[q * K + k];
    v[k] = r;
  }
}

// WPB windows per CTA: blockIdx.x = window group, blockIdx.z = pair - pair0.
// TH/TW/MY/MX: compile-time window and search sizes (SK) or 0 (RE).  CW = template columns
// per fp32 partial.  TMA: stage the search regions with cp.async.bulk.tensor; masks are read
// from global (L2) straight into the template-pair layout.  ALIAS: the score tile reuses the
// template-pair region (needs every item's scores in registers: items <= NT * IPT).
template <int TH, int TW, int MY, int MX, int RV, int CW, int NT, int WPB, int MINB, bool TMA, bool ALIAS, int IPT>
__global__ void __launch_bounds__(NT, MINB)
    piv_ncc_kernel(const PivArgs a, const __grid_constant__ CUtensorMap mapB) {
  constexpr bool SK = TH > 0;
  const PivShape<RV, CW> sh(SK ? TH : a.h, SK ? TW : a.w, SK ? MY : a.my, SK ? MX : a.mx,
                            SK ? piv_sk_pitch(TW, MX, RV, CW) : a.BP, ALIAS);
  extern __shared__ __align__(1024) unsigned char smem_raw[];
  float* smem = reinterpret_cast<float*>(smem_raw);
  constexpr int NW = (NT + 31) / 32;
  __shared__ double red[NW * 2 * WPB];
  __shared__ unsigned long long red_key[NW * WPB];
  __shared__ double s_energy[WPB], s_csum[WPB], s_mean[WPB], s_sumsq[WPB];
  __shared__ int s_flat[WPB];
  __shared__ __align__(8) uint64_t bar;

  const int tid = threadIdx.x;
  const int nwin = a.Ky * a.Kx;
  const int lz = blockIdx.z, pr = a.pair0 + lz;
  const int lin0 = blockIdx.x * WPB;
  const int nvalid = min(WPB, nwin - lin0);
  auto wy = [&](int wi) { return sh.my + ((lin0 + wi) / a.Kx) * a.sy; };
  auto wx = [&](int wi) { return sh.mx + ((lin0 + wi) % a.Kx) * a.sx; };
  auto TPw = [&](int wi) { return reinterpret_cast<u64*>(smem + wi * sh.win_fl + sh.tp_off()); };
  auto Bs = [&](int wi) { return smem + wi * sh.win_fl + sh.b_off(ALIAS); };
  auto Sc = [&](int wi) { return smem + wi * sh.win_fl + sh.s_off(ALIAS); };

  // ---- stage the search regions of frame B (TMA, or plain loads)
  if constexpr (TMA) {
    if (tid == 0) {
      tma_prefetch_desc(&mapB);
      mbar_init(&bar, 1);
      fence_mbar_init();
    }
    __syncthreads();
    if (tid == 0) {
      mbar_expect_tx(&bar, (uint32_t)(nvalid * sh.BR * sh.BP * 4));
      for (int wi = 0; wi < nvalid; ++wi) tma_load_3d(Bs(wi), &mapB, wx(wi) - sh.mx, wy(wi) - sh.my, pr, &bar);
    }
  } else {
    const float* Bf = a.B + (int64_t)pr * a.frame_stride;
    for (int wi = 0; wi < nvalid; ++wi) {
      float* bs = Bs(wi);
      const int by0 = wy(wi) - sh.my, bx0 = wx(wi) - sh.mx;
      for (int k = tid; k < sh.BR * sh.BP; k += NT) {
        const int i = k / sh.BP, j = k % sh.BP;
        const int gc = bx0 + j;
        bs[k] = gc < a.W ? __ldg(Bf + (int64_t)(by0 + i) * a.pitch + gc) : 0.0f;
      }
    }
  }

  // ---- mask statistics (Fig 5.2), masks read from global (L2): mean, A_D, sum of fp32 A_C;
  //      the centred mask is written straight into the template-pair layout.  Specialised
  //      kernels know the element count at compile time: each thread issues all its loads up
  //      front (latency overlapped) and keeps the values in registers for the second pass.
  const float* Af = a.A + (int64_t)pr * a.frame_stride;
  const int per_win = sh.h * sh.w;
  {
    constexpr int PERT = SK ? (WPB * TH * TW + NT - 1) / NT : 1;
    float mv[PERT];
    double v[2 * WPB];
#pragma unroll
    for (int q = 0; q < 2 * WPB; ++q) v[q] = 0.0;
    if constexpr (SK) {
#pragma unroll
      for (int k = 0; k < PERT; ++k) {
        const int e = tid + k * NT;
        const int wi = e / per_win, r = e % per_win;
        mv[k] = (wi < nvalid) ? __ldg(Af + (int64_t)(wy(wi) + r / sh.w) * a.pitch + wx(wi) + r % sh.w) : 0.0f;
      }
#pragma unroll
      for (int k = 0; k < PERT; ++k) {
        const int wi = (tid + k * NT) / per_win;
        const double t = mv[k];
#pragma unroll
        for (int q = 0; q < WPB; ++q)
          if (q == wi) { v[2 * q] += t; v[2 * q + 1] += t * t; }
      }
    } else {
      for (int e = tid; e < nvalid * per_win; e += NT) {
        const int wi = e / per_win, k = e % per_win;
        const double t = __ldg(Af + (int64_t)(wy(wi) + k / sh.w) * a.pitch + wx(wi) + k % sh.w);
#pragma unroll
        for (int q = 0; q < WPB; ++q)
          if (q == wi) { v[2 * q] += t; v[2 * q + 1] += t * t; }
      }
    }
    block_sum_k<2 * WPB>(v, red);
    const double n = (double)sh.h * (double)sh.w;
    double m[WPB], sumsq[WPB];
#pragma unroll
    for (int q = 0; q < WPB; ++q) { m[q] = v[2 * q] / n; sumsq[q] = v[2 * q + 1]; v[2 * q] = 0.0; v[2 * q + 1] = 0.0; }
    // centred value j of row i of window wi -> pairs TP[l].y and TP[l+1].x of its chunk
    auto put = [&](int wi, int i, int j, float ac) {
      float* tp = reinterpret_cast<float*>(TPw(wi) + i * sh.TPP + (j / CW) * sh.PB);
      const int l = j % CW;
      tp[2 * l + 1] = ac;
      tp[2 * (l + 1)] = ac;
      if (l == 0) tp[0] = 0.0f;               // TP[0].x = t[-1] = 0
      if (l == CW - 1) tp[2 * CW + 1] = 0.0f;  // TP[CW].y = t[CW] = 0
    };
    auto centre = [&](int wi, double x) {
      double mm = 0.0;
#pragma unroll
      for (int q = 0; q < WPB; ++q) mm = (q == wi) ? m[q] : mm;
      const double d = x - mm;
      const float ac = (float)d;
#pragma unroll
      for (int q = 0; q < WPB; ++q)
        if (q == wi) { v[2 * q] += d * d; v[2 * q + 1] += (double)ac; }
      return ac;
    };
    if constexpr (SK && (TW % CW == 0)) {  // no padding columns: every element is a mask value
#pragma unroll
      for (int k = 0; k < PERT; ++k) {
        const int e = tid + k * NT;
        const int wi = e / per_win, r = e % per_win;
        if (wi < nvalid) put(wi, r / sh.w, r % sh.w, centre(wi, (double)mv[k]));
      }
    } else {
      const int WPd = sh.nCW * CW;  // padded mask width
      const int per_pad = sh.h * WPd;
      for (int e = tid; e < nvalid * per_pad; e += NT) {
        const int wi = e / per_pad, k = e % per_pad;
        const int i = k / WPd, j = k % WPd;
        float ac = 0.0f;
        if (j < sh.w) ac = centre(wi, (double)__ldg(Af + (int64_t)(wy(wi) + i) * a.pitch + wx(wi) + j));
        put(wi, i, j, ac);
      }
    }
    block_sum_k<2 * WPB>(v, red);  // (its barriers also publish the template pairs)
    if (tid < WPB) {
      double e = 0, c = 0, ss = 0, mm = 0;
#pragma unroll
      for (int q = 0; q < WPB; ++q)
        if (q == tid) { e = v[2 * q]; c = v[2 * q + 1]; ss = sumsq[q]; mm = m[q]; }
      s_mean[tid] = mm;
      s_sumsq[tid] = ss;
      s_energy[tid] = e;
      s_csum[tid] = c;
      s_flat[tid] = (e <= kFlatRel * ss) ? 1 : 0;
    }
    if constexpr (TMA) mbar_wait(&bar, 0);
    __syncthreads();
  }

  // ---- numerator (FFMA2 pairs) over flattened items (window, row, group of RV shifts) + NCC
  const double inv_n = 1.0 / ((double)sh.h * (double)sh.w);
  const double* S1f = a.S1 + (int64_t)lz * a.map_frame_stride;
  const double* S2f = a.S2 + (int64_t)lz * a.map_frame_stride;
  const int nitems = nvalid * sh.items;
  float scv[ALIAS ? IPT : 1][RV];
#pragma unroll
  for (int k = 0; k < (ALIAS ? IPT : 1); ++k)
#pragma unroll
    for (int c = 0; c < RV; ++c) scv[k][c] = 0.0f;
  auto item = [&](int it, float (&out)[RV]) {
    const int wi = it / sh.items, r = it % sh.items;
    const int row = r / sh.NG, g = r % sh.NG;
    u64 tot2[RV / 2];
#pragma unroll
    for (int q = 0; q < RV / 2; ++q) tot2[q] = 0ull;
    const float* brow = Bs(wi) + row * sh.BP + g * RV;
    const u64* tpw = TPw(wi);
#pragma unroll 1
    for (int i = 0; i < sh.h; ++i) {
#pragma unroll 1
      for (int jc = 0; jc < sh.nCW; ++jc) {
        u64 part2[RV / 2];
#pragma unroll
        for (int q = 0; q < RV / 2; ++q) part2[q] = 0ull;
        row_dot_pairs<RV, CW>(brow + i * sh.BP + jc * CW, tpw + i * sh.TPP + jc * sh.PB, part2);
#pragma unroll
        for (int q = 0; q < RV / 2; ++q) add2(tot2[q], part2[q]);
      }
    }
    const double csum = s_csum[wi], energy = s_energy[wi];
    const bool flat = s_flat[wi] != 0;
    const int64_t mrow = (int64_t)(wy(wi) - sh.my + row) * a.map_pitch + (wx(wi) - sh.mx);
#pragma unroll
    for (int q = 0; q < RV / 2; ++q) {
      const float lo = __uint_as_float((uint32_t)(tot2[q] & 0xFFFFFFFFull));  // acc[2q+1]
      const float hi = __uint_as_float((uint32_t)(tot2[q] >> 32));           // acc[2q]
#pragma unroll
      for (int e = 0; e < 2; ++e) {
        const int c = 2 * q + 1 - e;
        const int col = g * RV + c;
        float s = 0.0f;
        if (col < sh.OX) {
          const double s1 = __ldg(S1f + mrow + col), s2 = __ldg(S2f + mrow + col);
          const float num = e == 0 ? lo : hi;
          s = a.ssd ? (float)(s_sumsq[wi] - 2.0 * ((double)num + s_mean[wi] * s1) + s2)
                    : ncc_normalize_fast(num, s1, s2, inv_n, csum, energy, flat);
        }
        out[c] = s;
      }
    }
    if constexpr (!ALIAS) {
      float* sc = Sc(wi) + row * sh.OXP + g * RV;
#pragma unroll
      for (int c = 0; c < RV; ++c) sc[c] = out[c];
    }
  };
  if constexpr (ALIAS) {
#pragma unroll
    for (int k = 0; k < IPT; ++k) {
      const int it = tid + k * NT;
      if (it < nitems) item(it, scv[k]);
    }
    __syncthreads();  // template pairs are dead: the score tile may overwrite them
#pragma unroll
    for (int k = 0; k < IPT; ++k) {
      const int it = tid + k * NT;
      if (it < nitems) {
        const int wi = it / sh.items, r = it % sh.items;
        float* sc = Sc(wi) + (r / sh.NG) * sh.OXP + (r % sh.NG) * RV;
#pragma unroll
        for (int c = 0; c < RV; ++c) sc[c] = scv[k][c];
      }
    }
  } else {
    for (int it = tid; it < nitems; it += NT) item(it, scv[0]);
  }
  __syncthreads();

  // ---- argmax per window (tie -> smallest row-major index), optional surface store
  const int tile = sh.OY * sh.OX;
  unsigned long long best[WPB];
#pragma unroll
  for (int q = 0; q < WPB; ++q) best[q] = 0ull;
  for (int e = tid; e < nvalid * tile; e += NT) {
    const int wi = e / tile, k = e % tile;
    const int row = k / sh.OX, col = k % sh.OX;
    const float s = Sc(wi)[row * sh.OXP + col];
    if (a.scores) a.scores[((int64_t)pr * nwin + lin0 + wi) * tile + k] = s;
    const unsigned long long key = make_key(a.ssd ? -s : s, (uint32_t)k);
#pragma unroll
    for (int q = 0; q < WPB; ++q)
      if (q == wi) best[q] = key > best[q] ? key : best[q];
  }
  {
    const int lane = tid & 31, wid = tid >> 5;
#pragma unroll
    for (int q = 0; q < WPB; ++q) best[q] = warp_max_key(best[q]);
    if (lane == 0) {
#pragma unroll
      for (int q = 0; q < WPB; ++q) red_key[wid * WPB + q] = best[q];
    }
    __syncthreads();
  }

  // ---- sub-pixel fit and the 24-B vector: one thread per window
  if (tid < nvalid) {
    const int wi = tid;
    unsigned long long bk = 0ull;
    for (int q = 0; q < NW; ++q) bk = red_key[q * WPB + wi] > bk ? red_key[q * WPB + wi] : bk;
    const float* S = Sc(wi);
    const uint32_t k = key_index(bk);
    const int row = (int)(k / sh.OX), col = (int)(k % sh.OX);
    const int iy = row - sh.my, ix = col - sh.mx;
    uint32_t flags = (s_flat[wi] && !a.ssd) ? (kFlatTemplate | kInvalid) : 0u;
    double ddy = 0.0, ddx = 0.0;
    bool par = false;
    if (row == 0 || row == sh.OY - 1) {
      flags |= kEdgeY;
    } else {
      const double cm = S[(row - 1) * sh.OXP + col], c0 = S[row * sh.OXP + col], cp = S[(row + 1) * sh.OXP + col];
      ddy = a.ssd ? subpix3_min(cm, c0, cp, a.subpix) : subpix3(cm, c0, cp, a.subpix, &par);
      if (par) flags |= kParabolaY;
    }
    if (col == 0 || col == sh.OX - 1) {
      flags |= kEdgeX;
    } else {
      const double cm = S[row * sh.OXP + col - 1], c0 = S[row * sh.OXP + col], cp = S[row * sh.OXP + col + 1];
      ddx = a.ssd ? subpix3_min(cm, c0, cp, a.subpix) : subpix3(cm, c0, cp, a.subpix, &par);
      if (par) flags |= kParabolaX;
    }
    VecOut o;
    o.iy = iy;
    o.ix = ix;
    o.dy = (float)(iy + ddy);
    o.dx = (float)(ix + ddx);
    o.score = a.ssd ? -key_score(bk) : key_score(bk);
    o.flags = flags;
    a.vec[(int64_t)pr * nwin + lin0 + wi] = o;
  }
}


// ================================================================== PIV, persistent + warp-specialised
// One CTA per SM loops over the windows of the launch.  NPW producer warps prepare window k+1
// (TMA of the search region, mask statistics, template pairs) and finish window k-1 (argmax,
// sub-pixel, vector store) while NCW consumer warps correlate window k -- the per-window
// prologue / epilogue that left the FMA pipe idle in piv_ncc_kernel is overlapped.
// Pipelines (mbarriers, parity = use index & 1):
//   full[s]  producer -> consumers: stage s (template pairs, B region, stats) ready
//   empty[s] consumers -> producer: stage s no longer read
//   scfull   consumers -> producer: score tile of window k written
//   scempty  producer -> consumers: score tile free again
template <int TH, int TW, int MY, int MX, int RV, int CW, int NCW, int NPW>
__global__ void __launch_bounds__((NCW + NPW) * 32, 1)
    piv_ws_kernel(const PivArgs a, const __grid_constant__ CUtensorMap mapB, int nwin_total) {
  constexpr int NCT = NCW * 32, NPT = NPW * 32;
  constexpr int BPc = piv_sk_pitch(TW, MX, RV, CW);
  const PivShape<RV, CW> sh(TH, TW, MY, MX, BPc, false);
  extern __shared__ __align__(1024) unsigned char smem_raw[];
  float* smem = reinterpret_cast<float*>(smem_raw);
  __shared__ __align__(8) uint64_t full_b[2], empty_b[2], scfull_b, scempty_b;
  __shared__ double st_mean[2], st_sumsq[2], st_energy[2], st_csum[2];
  __shared__ int st_flat[2];
  __shared__ double pred[NPW * 4];
  __shared__ unsigned long long pkey[NPW];
  auto TPs = [&](int s) { return reinterpret_cast<u64*>(smem + s * (sh.tp_fl + sh.b_fl)); };
  auto Bs = [&](int s) { return smem + s * (sh.tp_fl + sh.b_fl) + sh.tp_fl; };
  float* Sc = smem + 2 * (sh.tp_fl + sh.b_fl);

  const int tid = threadIdx.x;
  const int nwin = a.Ky * a.Kx;
  if (tid == 0) {
    tma_prefetch_desc(&mapB);
    mbar_init(&full_b[0], 2);
    mbar_init(&full_b[1], 2);
    mbar_init(&empty_b[0], NCT);
    mbar_init(&empty_b[1], NCT);
    mbar_init(&scfull_b, NCT);
    mbar_init(&scempty_b, 1);
    fence_mbar_init();
  }
  __syncthreads();
  const int nlocal = (nwin_total - (int)blockIdx.x + (int)gridDim.x - 1) / (int)gridDim.x;
  auto win_of = [&](int k, int& lz, int& lin) {
    const int wdx = (int)blockIdx.x + k * (int)gridDim.x;
    lz = wdx / nwin;
    lin = wdx % nwin;
  };

  if (tid >= NCT) {
    // =============================== producers
    const int pt = tid - NCT, lane = tid & 31, pw = pt >> 5;
    constexpr int PERT = (TH * TW + NPT - 1) / NPT;
    auto reduce2 = [&](double& x0, double& x1) {  // deterministic sum over the producer threads
      x0 = warp_sum_d(x0);
      x1 = warp_sum_d(x1);
      named_bar_sync(1, NPT);
      if (lane == 0) { pred[pw * 2] = x0; pred[pw * 2 + 1] = x1; }
      named_bar_sync(1, NPT);
      x0 = 0.0;
      x1 = 0.0;
      for (int q = 0; q < NPW; ++q) { x0 += pred[q * 2]; x1 += pred[q * 2 + 1]; }
    };
    auto epilogue = [&](int k) {
      int lz, lin;
      win_of(k, lz, lin);
      const int s = k & 1;
      mbar_wait_bounded(&scfull_b, (uint32_t)(k & 1));
      const int tile = sh.OY * sh.OX;
      unsigned long long best = 0ull;
      const int pr = a.pair0 + lz;
      for (int e = pt; e < tile; e += NPT) {
        const int row = e / sh.OX, col = e % sh.OX;
        const float sv = Sc[row * sh.OXP + col];
        if (a.scores) a.scores[((int64_t)pr * nwin + lin) * tile + e] = sv;
        const unsigned long long key = make_key(a.ssd ? -sv : sv, (uint32_t)e);
        best = key > best ? key : best;
      }
      best = warp_max_key(best);
      if (lane == 0) pkey[pw] = best;
      named_bar_sync(1, NPT);
      if (pt == 0) {
        unsigned long long bk = 0ull;
        for (int q = 0; q < NPW; ++q) bk = pkey[q] > bk ? pkey[q] : bk;
        const uint32_t kk = key_index(bk);
        const int row = (int)(kk / sh.OX), col = (int)(kk % sh.OX);
        const int iy = row - sh.my, ix = col - sh.mx;
        uint32_t flags = (st_flat[s] && !a.ssd) ? (kFlatTemplate | kInvalid) : 0u;
        double ddy = 0.0, ddx = 0.0;
        bool par = false;
        if (row == 0 || row == sh.OY - 1) {
          flags |= kEdgeY;
        } else {
          const double cm = Sc[(row - 1) * sh.OXP + col], c0 = Sc[row * sh.OXP + col],
                       cp = Sc[(row + 1) * sh.OXP + col];
          ddy = a.ssd ? subpix3_min(cm, c0, cp, a.subpix) : subpix3(cm, c0, cp, a.subpix, &par);
          if (par) flags |= kParabolaY;
        }
        par = false;
        if (col == 0 || col == sh.OX - 1) {
          flags |= kEdgeX;
        } else {
          const double cm = Sc[row * sh.OXP + col - 1], c0 = Sc[row * sh.OXP + col], cp = Sc[row * sh.OXP + col + 1];
          ddx = a.ssd ? subpix3_min(cm, c0, cp, a.subpix) : subpix3(cm, c0, cp, a.subpix, &par);
          if (par) flags |= kParabolaX;
        }
        VecOut o;
        o.iy = iy;
        o.ix = ix;
        o.dy = (float)(iy + ddy);
        o.dx = (float)(ix + ddx);
        o.score = a.ssd ? -key_score(bk) : key_score(bk);
        o.flags = flags;
        a.vec[(int64_t)pr * nwin + lin] = o;
        mbar_arrive(&scempty_b);  // the score tile may be overwritten
      }
      named_bar_sync(1, NPT);  // pkey / stats reuse
    };
    for (int k = 0; k < nlocal; ++k) {
      const int s = k & 1;
      int lz, lin;
      win_of(k, lz, lin);
      const int pr = a.pair0 + lz;
      const int y = sh.my + (lin / a.Kx) * a.sy, x = sh.mx + (lin % a.Kx) * a.sx;
      if (k >= 2) mbar_wait_bounded(&empty_b[s], (uint32_t)(((k >> 1) - 1) & 1));
      if (pt == 0) {
        mbar_expect_tx(&full_b[s], (uint32_t)(sh.BR * sh.BP * 4));
        tma_load_3d(Bs(s), &mapB, x - sh.mx, y - sh.my, pr, &full_b[s]);
      }
      // mask statistics and template pairs (as piv_ncc_kernel)
      const float* Af = a.A + (int64_t)pr * a.frame_stride;
      float mv[PERT];
#pragma unroll
      for (int q = 0; q < PERT; ++q) {
        const int e = pt + q * NPT;
        mv[q] = e < TH * TW ? __ldg(Af + (int64_t)(y + e / TW) * a.pitch + x + e % TW) : 0.0f;
      }
      double s1 = 0.0, s2 = 0.0;
#pragma unroll
      for (int q = 0; q < PERT; ++q) { s1 += (double)mv[q]; s2 += (double)mv[q] * (double)mv[q]; }
      reduce2(s1, s2);
      const double n = (double)TH * (double)TW;
      const double mean = s1 / n;
      double e2 = 0.0, cs = 0.0;
      u64* tpw = TPs(s);
#pragma unroll
      for (int q = 0; q < PERT; ++q) {
        const int e = pt + q * NPT;
        if (e < TH * TW) {
          const int i = e / TW, j = e % TW;
          const double d = (double)mv[q] - mean;
          const float ac = (float)d;
          e2 += d * d;
          cs += (double)ac;
          float* tp = reinterpret_cast<float*>(tpw + i * sh.TPP + (j / CW) * sh.PB);
          const int l = j % CW;
          tp[2 * l + 1] = ac;
          tp[2 * (l + 1)] = ac;
          if (l == 0) tp[0] = 0.0f;
          if (l == CW - 1) tp[2 * CW + 1] = 0.0f;
        }
      }
      reduce2(e2, cs);
      if (pt == 0) {
        st_mean[s] = mean;
        st_sumsq[s] = s2;
        st_energy[s] = e2;
        st_csum[s] = cs;
        st_flat[s] = (e2 <= kFlatRel * s2) ? 1 : 0;
      }
      named_bar_sync(1, NPT);  // template pairs + stats of all producers written
      if (pt == 0) mbar_arrive(&full_b[s]);
      if (k >= 1) epilogue(k - 1);
    }
    if (nlocal >= 1) epilogue(nlocal - 1);
  } else {
    // =============================== consumers
    const int ct = tid;
    const bool has = ct < sh.items;
    const int row = has ? ct / sh.NG : 0, g = has ? ct % sh.NG : 0;
    const double inv_n = 1.0 / ((double)TH * (double)TW);
    for (int k = 0; k < nlocal; ++k) {
      const int s = k & 1;
      int lz, lin;
      win_of(k, lz, lin);
      const int y = sh.my + (lin / a.Kx) * a.sy, x = sh.mx + (lin % a.Kx) * a.sx;
      mbar_wait_bounded(&full_b[s], (uint32_t)((k >> 1) & 1));
      float out[RV];
      if (has) {
        u64 tot2[RV / 2];
#pragma unroll
        for (int q = 0; q < RV / 2; ++q) tot2[q] = 0ull;
        const float* brow = Bs(s) + row * sh.BP + g * RV;
        const u64* tpw = TPs(s);
#pragma unroll 1
        for (int i = 0; i < TH; ++i) {
#pragma unroll
          for (int jc = 0; jc < (TW + CW - 1) / CW; ++jc) {
            u64 part2[RV / 2];
#pragma unroll
            for (int q = 0; q < RV / 2; ++q) part2[q] = 0ull;
            row_dot_pairs<RV, CW>(brow + i * sh.BP + jc * CW, tpw + i * sh.TPP + jc * sh.PB, part2);
#pragma unroll
            for (int q = 0; q < RV / 2; ++q) add2(tot2[q], part2[q]);
          }
        }
        const double csum = st_csum[s], energy = st_energy[s], tmean = st_mean[s], tsq = st_sumsq[s];
        const bool flat = st_flat[s] != 0;
        const double* S1f = a.S1 + (int64_t)lz * a.map_frame_stride;
        const double* S2f = a.S2 + (int64_t)lz * a.map_frame_stride;
        const int64_t mrow = (int64_t)(y - sh.my + row) * a.map_pitch + (x - sh.mx);
#pragma unroll
        for (int q = 0; q < RV / 2; ++q) {
          const float lo = __uint_as_float((uint32_t)(tot2[q] & 0xFFFFFFFFull));
          const float hi = __uint_as_float((uint32_t)(tot2[q] >> 32));
#pragma unroll
          for (int e = 0; e < 2; ++e) {
            const int c = 2 * q + 1 - e;
            const int col = g * RV + c;
            float v = 0.0f;
            if (col < sh.OX) {
              const double s1 = __ldg(S1f + mrow + col), s2 = __ldg(S2f + mrow + col);
              const float num = e == 0 ? lo : hi;
              v = a.ssd ? (float)(tsq - 2.0 * ((double)num + tmean * s1) + s2)
                        : ncc_normalize_fast(num, s1, s2, inv_n, csum, energy, flat);
            }
            out[c] = v;
          }
        }
      }
      mbar_arrive(&empty_b[s]);  // done reading stage s (pairs, region, stats)
      if (k >= 1) mbar_wait_bounded(&scempty_b, (uint32_t)((k - 1) & 1));
      if (has) {
        float* sc = Sc + row * sh.OXP + g * RV;
#pragma unroll
        for (int c = 0; c < RV; ++c) sc[c] = out[c];
      }
      mbar_arrive(&scfull_b);
    }
  }
}

// Sum of v[i] over the 32 lanes of a warp, for all 32 i at once: each level keeps half of the
// values and swaps the other half with the partner lane (16 + 8 + 4 + 2 + 1 shuffles); lane l
// ends with the total of v[l].
__device__ __forceinline__ float warp_transpose_sum32(float (&v)[32]) {
  const int lane = threadIdx.x & 31;
#pragma unroll
  for (int d = 16; d >= 1; d >>= 1) {
    const bool up = (lane & d) != 0;
#pragma unroll
    for (int i = 0; i < d; ++i) {
      const float send = up ? v[i] : v[i + d];
      const float keep = up ? v[i + d] : v[i];
      v[i] = keep + __shfl_xor_sync(0xffffffffu, send, d);
    }
  }
  return v[0];
}

// ================================================================== PIV, persistent + warp-specialised, balanced core
// piv_ws_kernel spreads (2m+1) x ceil((2m+1)/RV) items over 13 consumer warps: the SMSP that
// holds 4 of them sets the pace (13/16 of the FMA pipe) and 7 of every 72 columns are padding.
// Here the consumers own exactly the 2m_y x 2m_x core of each offset grid -- NCW warps, two
// per SMSP, RV = 16 shifts per lane, no padding -- and the producer warps, otherwise idle while
// a window is correlated, compute the (2m_x+1) + 2m_y border offsets (last row dy = +m_y, last
// column dx = +m_x) from the same staged stage.  A stage holds WPS windows (cfg 4: one 64x64
// window; cfg 3: four 32x32 windows) so that every consumer lane owns RV core offsets.
// Consumer lane layout: each 8-lane LDS.128 phase covers 4 rows x 2 column groups and the
// staged pitch (BP = 4 mod 32 floats) puts them on 8 distinct 16-B bank groups.
__host__ __device__ constexpr int piv_ws2_pitch(int TW, int MX, int CW) {
  return (((2 * MX + ((TW + CW - 1) / CW) * CW) - 4 + 31) / 32) * 32 + 4;
}
template <int TH, int TW, int MY, int MX, int RV, int CW, int WPS>
struct PivWs2Shape {
  static constexpr int OY = 2 * MY + 1, OX = 2 * MX + 1, OYc = 2 * MY, OXc = 2 * MX, NG = OXc / RV;
  static constexpr int nCW = TW / CW, PB = CW + 2, TPP = nCW * PB, BR = TH + 2 * MY;
  static constexpr int BP = piv_ws2_pitch(TW, MX, CW);
  static constexpr int SP = (OX + 3) & ~3;  // score tile pitch
  static constexpr int tp_fl = ((TH * TPP * 2 + 31) / 32) * 32, b_fl = ((BR * BP + 31) / 32) * 32;
  static constexpr int s_fl = ((OY * SP + 31) / 32) * 32;
  static constexpr int stage_fl = WPS * (tp_fl + b_fl);
  static constexpr int NE = OX + OYc;      // border offsets of one window (producers)
  static constexpr int RPW = 32 / NG;      // core rows per consumer warp
  static constexpr int WPW = OYc / RPW;    // consumer warps per window
  static constexpr int smem_bytes = (2 * stage_fl + WPS * s_fl) * 4;
};
#ifdef NCC_PIV_TRACE  // tools/microbench/piv_trace.cu: clock64 stamps per stage of CTA 0
__device__ long long* g_piv_trace;
#define PIV_STAMP(slot, k) \
  if (blockIdx.x == 0 && (k) < 64) g_piv_trace[(slot)*64 + (k)] = clock64()
__device__ int g_piv_exp;  // timing experiments (trace builds only): 1 no border sums, 2 no epilogue normalisation
#define PIV_EXP(bit) (g_piv_exp & (bit))
#else
#define PIV_STAMP(slot, k)
#define PIV_EXP(bit) 0
#endif
template <int TH, int TW, int MY, int MX, int RV, int CW, int NCW, int NPW, int WPS>
__global__ void __launch_bounds__((NCW + NPW) * 32, 1)
    piv_ws2_kernel(const PivArgs a, const __grid_constant__ CUtensorMap mapB, int nwin_total) {
  using S = PivWs2Shape<TH, TW, MY, MX, RV, CW, WPS>;
  constexpr int NCT = NCW * 32, NPT = NPW * 32;
  static_assert(RV == 16 && S::OXc % RV == 0 && (S::NG == 2 || S::NG == 4), "lane layout: 2 or 4 groups per row");
  static_assert(S::OYc % S::RPW == 0 && S::WPW * WPS == NCW, "consumer warps tile the cores of the stage");
  static_assert(TW % CW == 0 && CW % 4 == 0 && TW % 32 == 0, "whole column chunks and 32-column lane strips");
  static_assert((S::BP / 4) % 8 == 1, "conflict-free LDS.128 phases");
  static_assert(WPS <= NPW && NPW % WPS == 0, "producer warps split evenly over the windows of a stage");
  constexpr int PPW = NPW / WPS;                        // producer warps per window (border offsets)
  constexpr int NEW = (S::NE + PPW - 1) / PPW;          // border offsets per producer warp
  constexpr int EPT = (NEW + 31) / 32;                  // ... per lane
  constexpr int JPL = TW / 32;                          // template columns per lane (border sums)
  // Register-reusing border sums: half of a window's producer warps take the last row
  // (dy = 2m_y), each a 16-offset slice dx0 = 16 w (the last slice up to 2m_x + 1), lane = template
  // row (mod 32), sliding along the staged image row in chunks of JC template columns; the other
  // half take the last column (dx = 2m_x) in 16-offset slices of dy, lane = template column (mod
  // 32), sliding down the staged image column in chunks of IC template rows.  Each staged value
  // feeds 16-33 products (the scalar form loaded one value per product: half of a stage's
  // shared-memory traffic, which stalled the consumers' LDS.128 stream).  A transpose-sum over
  // the lanes leaves offset o of the slice in lane o.
  constexpr int RWb = PPW / 2, CWb = PPW / 2;                     // row / column border warps
  constexpr int AX = S::OX - 16 * (RWb - 1), AY = S::OYc - 16 * (CWb - 1);  // last slices' sizes
  constexpr int RPL = (TH + 31) / 32, CPL = (TW + 31) / 32;        // template rows / columns per lane
  constexpr int JC = TW <= 32 ? TW : 16, IC = TH <= 32 ? TH : 16;  // chunk of template columns / rows
  constexpr bool kRB = PPW % 2 == 0 && PPW >= 2 && AX >= 16 && AX <= 33 && (AX < 33 || EPT >= 2) && AY >= 1 &&
                       AY <= 32 && TW % JC == 0 &&
                       TH % IC == 0 && JC % 4 == 0 && (TH <= 32 || TH % 32 == 0) && (TW <= 32 || TW % 32 == 0);
  static_assert((TH * TW) % NPT == 0 && NPT % TW == 0, "producer threads tile each mask in whole rows");
  extern __shared__ __align__(1024) unsigned char smem_raw[];
  float* smem = reinterpret_cast<float*>(smem_raw);
  __shared__ __align__(8) uint64_t full_b[2], empty_b[2], scfull_b, scempty_b;
  __shared__ double st_mean[2][WPS], st_sumsq[2][WPS], st_energy[2][WPS], st_csum[2][WPS];
  __shared__ int st_flat[2][WPS];
  __shared__ double pred[NPW * 2 * WPS];
  __shared__ unsigned long long pkey[NPW][WPS];
  auto TPs = [&](int s, int wi) { return reinterpret_cast<u64*>(smem + s * S::stage_fl + wi * S::tp_fl); };
  auto Bs = [&](int s, int wi) { return smem + s * S::stage_fl + WPS * S::tp_fl + wi * S::b_fl; };
  auto Sc = [&](int wi) { return smem + 2 * S::stage_fl + wi * S::s_fl; };

  const int tid = threadIdx.x;
  const int nwin = a.Ky * a.Kx;
  if (tid == 0) {
    tma_prefetch_desc(&mapB);
    mbar_init(&full_b[0], 2);
    mbar_init(&full_b[1], 2);
    mbar_init(&empty_b[0], NCT);
    mbar_init(&empty_b[1], NCT);
    mbar_init(&scfull_b, NCT);
    mbar_init(&scempty_b, 1);
    fence_mbar_init();
  }
  __syncthreads();
  // Windows are dealt to the CTAs one at a time (CTA c: windows c, c + G, c + 2G, ...), so the
  // CTAs' window counts differ by at most one and only their LAST stage is partly filled: at
  // cfg 3 (3,721 windows, 148 CTAs, 4 per stage) every CTA runs 6 full stages + one of 1-2
  // windows, instead of 43 CTAs running a 7th full stage while the others idle.
  const int nmine = (nwin_total - (int)blockIdx.x + (int)gridDim.x - 1) / (int)gridDim.x;
  const int nlocal = (nmine + WPS - 1) / WPS;
  // window wi of the k-th stage of this CTA: pair (relative to pair0) and linear index
  auto win_of = [&](int k, int wi, int& lz, int& lin) {
    const int j = k * WPS + wi;
    const int wdx = (int)blockIdx.x + j * (int)gridDim.x;
    lz = wdx / nwin;
    lin = wdx % nwin;
    return j < nmine;
  };
  const double inv_n = 1.0 / ((double)TH * (double)TW);

  if (tid >= NCT) {
    // =============================== producers
    const int pt = tid - NCT, lane = tid & 31, pw = pt >> 5;
    const int bwin = pw / PPW, bsub = pw % PPW;  // this warp's border window and its offset stride slot
    constexpr int PERT = (WPS * TH * TW + NPT - 1) / NPT;
    auto border = [&](int e, int& dy, int& dx) {
      if (e < S::OX) { dy = S::OYc; dx = e; } else { dy = e - S::OX; dx = S::OXc; }
    };
    auto owned = [&](int q) { return bsub + PPW * (lane + 32 * q); };  // border offset of slot q
    float ext_prev[EPT];
    auto epilogue = [&](int k) {
      mbar_wait_backoff(&scfull_b, (uint32_t)(k & 1));
      if (pt == 0) PIV_STAMP(6, k);
      const int s = k & 1;
      if constexpr (kRB) {  // row warp w: lane o -> (2m_y, 16 w + o) [+ the 33rd in lane 0];
                            // column warp w: lane o -> (16 w + o, 2m_x)
        if (bsub < RWb) {
          const int n = bsub == RWb - 1 ? AX : 16;
          if (lane < n && lane < 32) Sc(bwin)[S::OYc * S::SP + 16 * bsub + lane] = ext_prev[0];
          if (n == 33 && lane == 0) Sc(bwin)[S::OYc * S::SP + 16 * bsub + 32] = ext_prev[EPT - 1];
        } else {
          const int w = bsub - RWb, n = w == CWb - 1 ? AY : 16;
          if (lane < n) Sc(bwin)[(16 * w + lane) * S::SP + S::OXc] = ext_prev[0];
        }
      } else {
#pragma unroll
        for (int q = 0; q < EPT; ++q) {  // border scores of group k (computed during its core)
          const int e = owned(q);
          if (e < S::NE) {
            int dy, dx;
            border(e, dy, dx);
            Sc(bwin)[dy * S::SP + dx] = ext_prev[q];
          }
        }
      }
      named_bar_sync(1, NPT);
      // normalise every offset of the stage's windows (numerators -> NCC / SSD from the fp64
      // window sums), write the scores back for the sub-pixel fit, per-window argmax keys
      constexpr int tile = S::OY * S::OX;
      constexpr int CH = 8;  // window-sum loads in flight per thread
      unsigned long long best[WPS];
#pragma unroll
      for (int wi = 0; wi < WPS; ++wi) {
        best[wi] = 0ull;
        int lz, lin;
        if (!win_of(k, wi, lz, lin)) continue;
        const int y0 = (lin / a.Kx) * a.sy, x0 = (lin % a.Kx) * a.sx;  // map origin (y - m_y, x - m_x)
        const double* S1f = a.S1 + (int64_t)lz * a.map_frame_stride + (int64_t)y0 * a.map_pitch + x0;
        const double* S2f = a.S2 + (int64_t)lz * a.map_frame_stride + (int64_t)y0 * a.map_pitch + x0;
        const double csum = st_csum[s][wi], energy = st_energy[s][wi], tmean = st_mean[s][wi],
                     tsq = st_sumsq[s][wi];
        const bool flat = st_flat[s][wi] != 0;
        float* T = Sc(wi);
        float* gsc = a.scores ? a.scores + ((int64_t)(a.pair0 + lz) * nwin + lin) * tile : nullptr;
        unsigned long long bw = 0ull;
        // NCC from the window kernel's fp32 factors (rsqrt(n var), S1/n; fp64-derived, rounded
        // once): three fp32 roundings per score instead of fp64 loads and arithmetic
        const bool fac = a.rsv != nullptr && !a.ssd;
        const float* RVf = fac ? a.rsv + (S1f - a.S1) : nullptr;
        const float* MNf = fac ? a.mean + (S1f - a.S1) : nullptr;
        const float csf = (float)csum, rse = flat ? 0.0f : (float)(1.0 / sqrt(energy));
        for (int e0 = pt; e0 < tile; e0 += CH * NPT) {
          double w1[CH], w2[CH];
          float f1[CH], f2[CH];
#pragma unroll
          for (int c = 0; c < CH; ++c) {
            const int e = e0 + c * NPT;
            if (e < tile && !PIV_EXP(2)) {
              const int64_t mi = (int64_t)(e / S::OX) * a.map_pitch + e % S::OX;
              if (fac) {
                f1[c] = __ldg(RVf + mi);
                f2[c] = __ldg(MNf + mi);
              } else {
                w1[c] = __ldg(S1f + mi);
                w2[c] = __ldg(S2f + mi);
              }
            }
          }
#pragma unroll
          for (int c = 0; c < CH; ++c) {
            const int e = e0 + c * NPT;
            if (e < tile) {
              float* tp = T + (e / S::OX) * S::SP + e % S::OX;
              const float num = *tp;
              float sv;
              if (PIV_EXP(2)) {
                sv = num;
              } else if (fac) {
                const float r = fmaf(-csf, f2[c], num) * (f1[c] * rse);
                sv = r > 1.0f ? 1.0f : (r < -1.0f ? -1.0f : r);
              } else {
                sv = a.ssd ? (float)(tsq - 2.0 * ((double)num + tmean * w1[c]) + w2[c])
                           : ncc_normalize_fast(num, w1[c], w2[c], inv_n, csum, energy, flat);
              }
              *tp = sv;
              if (gsc) gsc[e] = sv;
              const unsigned long long key = make_key(a.ssd ? -sv : sv, (uint32_t)e);
              bw = key > bw ? key : bw;
            }
          }
        }
        best[wi] = bw;
      }
#pragma unroll
      for (int wi = 0; wi < WPS; ++wi) {
        best[wi] = warp_max_key(best[wi]);
        if (lane == 0) pkey[pw][wi] = best[wi];
      }
      named_bar_sync(1, NPT);
      if (pt < WPS) {
        const int wi = pt;
        int lz, lin;
        if (win_of(k, wi, lz, lin)) {
          const float* T = Sc(wi);
          unsigned long long bk = 0ull;
          for (int q = 0; q < NPW; ++q) bk = pkey[q][wi] > bk ? pkey[q][wi] : bk;
          const uint32_t kk = key_index(bk);
          const int row = (int)(kk / S::OX), col = (int)(kk % S::OX);
          const int iy = row - MY, ix = col - MX;
          uint32_t flags = (st_flat[s][wi] && !a.ssd) ? (kFlatTemplate | kInvalid) : 0u;
          double ddy = 0.0, ddx = 0.0;
          bool par = false;
          if (row == 0 || row == S::OY - 1) {
            flags |= kEdgeY;
          } else {
            const double cm = T[(row - 1) * S::SP + col], c0 = T[row * S::SP + col], cp = T[(row + 1) * S::SP + col];
            ddy = a.ssd ? subpix3_min(cm, c0, cp, a.subpix) : subpix3(cm, c0, cp, a.subpix, &par);
            if (par) flags |= kParabolaY;
          }
          par = false;
          if (col == 0 || col == S::OX - 1) {
            flags |= kEdgeX;
          } else {
            const double cm = T[row * S::SP + col - 1], c0 = T[row * S::SP + col], cp = T[row * S::SP + col + 1];
            ddx = a.ssd ? subpix3_min(cm, c0, cp, a.subpix) : subpix3(cm, c0, cp, a.subpix, &par);
            if (par) flags |= kParabolaX;
          }
          VecOut o;
          o.iy = iy;
          o.ix = ix;
          o.dy = (float)(iy + ddy);
          o.dx = (float)(ix + ddx);
          o.score = a.ssd ? -key_score(bk) : key_score(bk);
          o.flags = flags;
          a.vec[(int64_t)(a.pair0 + lz) * nwin + lin] = o;
        }
      }
      named_bar_sync(1, NPT);  // every score tile read; pkey / stats reusable
      if (pt == 0) mbar_arrive(&scempty_b);  // the score tiles may be overwritten
      if (pt == 0) PIV_STAMP(7, k);
    };
    for (int k = 0; k < nlocal; ++k) {
      const int s = k & 1;
      int wy[WPS], wx[WPS], wz[WPS];
      bool wv[WPS];
      int nvalid = 0;
#pragma unroll
      for (int wi = 0; wi < WPS; ++wi) {
        int lz, lin;
        wv[wi] = win_of(k, wi, lz, lin);
        wz[wi] = a.pair0 + lz;
        wy[wi] = MY + (lin / a.Kx) * a.sy;
        wx[wi] = MX + (lin % a.Kx) * a.sx;
        nvalid += wv[wi] ? 1 : 0;
      }
      if (pt == 0) PIV_STAMP(0, k);
      if (k >= 2) mbar_wait_bounded(&empty_b[s], (uint32_t)(((k >> 1) - 1) & 1));
      if (pt == 0) PIV_STAMP(1, k);
      if (pt == 0) {
        mbar_expect_tx(&full_b[s], (uint32_t)(nvalid * S::BR * S::BP * 4));
#pragma unroll
        for (int wi = 0; wi < WPS; ++wi)
          if (wv[wi]) tma_load_3d(Bs(s, wi), &mapB, wx[wi] - MX, wy[wi] - MY, wz[wi], &full_b[s]);
      }
      // mask statistics (Fig 5.2) and template pairs, all windows of the stage at once; element
      // pt + q*NPT of the stage = window q / QPW, row pt / TW + (q % QPW) * RPQ, column pt % TW
      constexpr int QPW = TH * TW / NPT, RPQ = NPT / TW;
      const int pr0 = pt / TW, pc0 = pt % TW;
      float mv[PERT];
#pragma unroll
      for (int wi = 0; wi < WPS; ++wi) {
        const float* Aw = a.A + (int64_t)wz[wi] * a.frame_stride + (int64_t)(wy[wi] + pr0) * a.pitch + wx[wi] + pc0;
#pragma unroll
        for (int q = 0; q < QPW; ++q) mv[wi * QPW + q] = wv[wi] ? __ldg(Aw + (int64_t)(q * RPQ) * a.pitch) : 0.0f;
      }
      double v[2 * WPS];
#pragma unroll
      for (int wi = 0; wi < 2 * WPS; ++wi) v[wi] = 0.0;
#pragma unroll
      for (int q = 0; q < PERT; ++q) {
        const int wi = q / QPW;
        const double t = (double)mv[q];
#pragma unroll
        for (int w2 = 0; w2 < WPS; ++w2)
          if (w2 == wi) { v[2 * w2] += t; v[2 * w2 + 1] += t * t; }
      }
      auto reduce = [&]() {  // deterministic sums over the producer threads
#pragma unroll
        for (int j = 0; j < 2 * WPS; ++j) v[j] = warp_sum_d(v[j]);
        named_bar_sync(1, NPT);
        if (lane == 0)
#pragma unroll
          for (int j = 0; j < 2 * WPS; ++j) pred[pw * 2 * WPS + j] = v[j];
        named_bar_sync(1, NPT);
#pragma unroll
        for (int j = 0; j < 2 * WPS; ++j) {
          double r = 0.0;
          for (int q = 0; q < NPW; ++q) r += pred[q * 2 * WPS + j];
          v[j] = r;
        }
      };
      reduce();
      if (pt == 0) PIV_STAMP(2, k);
      double mean[WPS], sumsq[WPS];
#pragma unroll
      for (int wi = 0; wi < WPS; ++wi) {
        mean[wi] = v[2 * wi] * inv_n;
        sumsq[wi] = v[2 * wi + 1];
        v[2 * wi] = 0.0;
        v[2 * wi + 1] = 0.0;
      }
#pragma unroll
      for (int q = 0; q < PERT; ++q) {
        const int wi = q / QPW, i = pr0 + (q % QPW) * RPQ, j = pc0;
        double mm = 0.0;
#pragma unroll
        for (int w2 = 0; w2 < WPS; ++w2) mm = (w2 == wi) ? mean[w2] : mm;
        const double d = (double)mv[q] - mm;
        const float ac = (float)d;
#pragma unroll
        for (int w2 = 0; w2 < WPS; ++w2)
          if (w2 == wi) { v[2 * w2] += d * d; v[2 * w2 + 1] += (double)ac; }
        float* tp = reinterpret_cast<float*>(TPs(s, wi) + i * S::TPP + (j / CW) * S::PB);
        const int l = j % CW;
        tp[2 * l + 1] = ac;
        tp[2 * (l + 1)] = ac;
        if (l == 0) tp[0] = 0.0f;
        if (l == CW - 1) tp[2 * CW + 1] = 0.0f;
      }
      reduce();
      if (pt < WPS) {
        double mm = 0, ss = 0, ee = 0, cc = 0;
#pragma unroll
        for (int w2 = 0; w2 < WPS; ++w2)
          if (w2 == pt) { mm = mean[w2]; ss = sumsq[w2]; ee = v[2 * w2]; cc = v[2 * w2 + 1]; }
        st_mean[s][pt] = mm;
        st_sumsq[s][pt] = ss;
        st_energy[s][pt] = ee;
        st_csum[s][pt] = cc;
        st_flat[s][pt] = (ee <= kFlatRel * ss) ? 1 : 0;
      }
      named_bar_sync(1, NPT);  // template pairs + stats of all producers written
      if (pt == 0) mbar_arrive(&full_b[s]);
      if (pt == 0) PIV_STAMP(3, k);
      // Border offsets of this warp's window: lanes split the template columns (j = lane + 32c),
      // the warp walks up to 32 offsets per pass; conflict-free scalar loads of the region, the
      // template value loaded once per row; per-lane fp32 sums over <= JPL*TH products, then a
      // butterfly sum across the lanes.
      mbar_wait_bounded(&full_b[s], (uint32_t)((k >> 1) & 1));  // search regions landed
      if (pt == 0) PIV_STAMP(4, k);
      float ext_cur[EPT];
#pragma unroll
      for (int q = 0; q < EPT; ++q) ext_cur[q] = 0.0f;
      bool bvalid = false;
#pragma unroll
      for (int w2 = 0; w2 < WPS; ++w2) bvalid = (w2 == bwin) ? wv[w2] : bvalid;
      if (PIV_EXP(1)) {
      } else if (kRB && bvalid) {
        const float* tpf = reinterpret_cast<const float*>(TPs(s, bwin));
        auto tval = [&](int i, int j) { return tpf[(i * S::TPP + (j / CW) * S::PB) * 2 + 1 + 2 * (j % CW)]; };
        const float* bsr = Bs(s, bwin);
        float blk[32];
        if (bsub < RWb) {
          // last row, slice dx in [dx0, dx0 + n): out[dx] = sum_i sum_j T[i][j] B[i + 2m_y][j + dx]
          const int dx0 = 16 * bsub;
          float acc[AX];
#pragma unroll
          for (int d = 0; d < AX; ++d) acc[d] = 0.0f;
#pragma unroll
          for (int ri = 0; ri < RPL; ++ri) {
            const int i = lane + 32 * ri;
            if (i < TH) {
              const float* brow = bsr + (i + S::OYc) * S::BP + dx0;
#pragma unroll 1
              for (int j0 = 0; j0 < TW; j0 += JC) {
                float t[JC];
#pragma unroll
                for (int j = 0; j < JC; ++j) t[j] = tval(i, j0 + j);
#pragma unroll
                for (int c4 = 0; c4 < JC + AX - 1; c4 += 4) {
                  const float4 v = *reinterpret_cast<const float4*>(brow + j0 + c4);
                  const float b[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
                  for (int e = 0; e < 4; ++e)
#pragma unroll
                    for (int d = 0; d < AX; ++d) {
                      const int j = c4 + e - d;
                      if (j >= 0 && j < JC) acc[d] = fmaf(t[j], b[e], acc[d]);
                    }
                }
              }
            }
          }
#pragma unroll
          for (int d = 0; d < 32; ++d) blk[d] = d < AX ? acc[d] : 0.0f;
          ext_cur[0] = warp_transpose_sum32(blk);
          if constexpr (AX == 33) {  // the 33rd offset of the slice: plain warp sum into lane 0
            float x = acc[AX - 1];
#pragma unroll
            for (int o = 16; o; o >>= 1) x += __shfl_xor_sync(0xffffffffu, x, o);
            ext_cur[EPT - 1] = lane == 0 ? x : ext_cur[EPT - 1];
          }
        } else {
          // last column, slice dy in [dy0, dy0 + n): out[dy] = sum_i sum_j T[i][j] B[i + dy][j + 2m_x]
          const int dy0 = 16 * (bsub - RWb);
          float acc[AY];
#pragma unroll
          for (int d = 0; d < AY; ++d) acc[d] = 0.0f;
#pragma unroll
          for (int cj = 0; cj < CPL; ++cj) {
            const int j = lane + 32 * cj;
            if (j < TW) {
              const float* bcol = bsr + dy0 * S::BP + S::OXc + j;
#pragma unroll 1
              for (int i0 = 0; i0 < TH; i0 += IC) {
                float t[IC];
#pragma unroll
                for (int i = 0; i < IC; ++i) t[i] = tval(i0 + i, j);
#pragma unroll
                for (int r8 = 0; r8 < IC + AY - 1; r8 += 8) {
                  float b[8];
#pragma unroll
                  for (int e = 0; e < 8; ++e) b[e] = r8 + e < IC + AY - 1 ? bcol[(i0 + r8 + e) * S::BP] : 0.0f;
#pragma unroll
                  for (int e = 0; e < 8; ++e)
#pragma unroll
                    for (int d = 0; d < AY; ++d) {
                      const int i = r8 + e - d;
                      if (i >= 0 && i < IC) acc[d] = fmaf(t[i], b[e], acc[d]);
                    }
                }
              }
            }
          }
#pragma unroll
          for (int d = 0; d < 32; ++d) blk[d] = d < AY ? acc[d] : 0.0f;
          ext_cur[0] = warp_transpose_sum32(blk);
        }
      } else if (bvalid) {
        const float* tpf = reinterpret_cast<const float*>(TPs(s, bwin));
        const float* bs = Bs(s, bwin) + lane;
        // one pass over the rows for all NEW offsets of the warp (offsets past NE compute
        // harmless products from the staged region and are dropped)
        int boff[NEW];
#pragma unroll
        for (int o = 0; o < NEW; ++o) {
          const int e = bsub + PPW * o;
          int dy = 0, dx = 0;
          if (e < S::NE) border(e, dy, dx);
          boff[o] = dy * S::BP + dx;
        }
        float acc[EPT * 32];
#pragma unroll
        for (int o = 0; o < EPT * 32; ++o) acc[o] = 0.0f;
#pragma unroll 1
        for (int i = 0; i < TH; ++i) {
          float tv[JPL];
#pragma unroll
          for (int c = 0; c < JPL; ++c) {
            const int j = lane + 32 * c;
            tv[c] = tpf[(i * S::TPP + (j / CW) * S::PB) * 2 + 1 + 2 * (j % CW)];
          }
          const float* br = bs + i * S::BP;
#pragma unroll
          for (int o = 0; o < NEW; ++o)
#pragma unroll
            for (int c = 0; c < JPL; ++c) acc[o] = fmaf(tv[c], br[boff[o] + 32 * c], acc[o]);
        }
#pragma unroll
        for (int q = 0; q < EPT; ++q) {
          float blk[32];
#pragma unroll
          for (int o = 0; o < 32; ++o) blk[o] = acc[32 * q + o];
          ext_cur[q] = warp_transpose_sum32(blk);  // raw numerator of offset owned(q)
        }
      }
      if (pt == 0) PIV_STAMP(5, k);
      if (k >= 1) epilogue(k - 1);
#pragma unroll
      for (int q = 0; q < EPT; ++q) ext_prev[q] = ext_cur[q];
    }
    if (nlocal >= 1) epilogue(nlocal - 1);
  } else {
    // =============================== consumers: RPW core rows x NG groups of RV shifts per warp
    const int wq = tid >> 5, l = tid & 31, ph = l >> 3, q8 = l & 7;
    constexpr int PHR = S::NG / 2;  // 8-lane phases per 4-row block
    const int wi = wq / S::WPW;
    const int row = (wq % S::WPW) * S::RPW + 4 * (ph / PHR) + (q8 & 3);
    const int g = (q8 >> 2) + 2 * (ph % PHR);
    for (int k = 0; k < nlocal; ++k) {
      const int s = k & 1;
      int lz, lin;
      const bool valid = win_of(k, wi, lz, lin);
      mbar_wait_bounded(&full_b[s], (uint32_t)((k >> 1) & 1));
      if (tid == 0) PIV_STAMP(8, k);
      float out[RV];
#pragma unroll
      for (int c = 0; c < RV; ++c) out[c] = 0.0f;
      if (valid) {
        u64 tot2[RV / 2];
#pragma unroll
        for (int q = 0; q < RV / 2; ++q) tot2[q] = 0ull;
        const float* brow = Bs(s, wi) + row * S::BP + g * RV;
        const u64* tpw = TPs(s, wi);
#pragma unroll 2
        for (int i = 0; i < TH; ++i) {
#pragma unroll
          for (int jc = 0; jc < S::nCW; ++jc) {
            u64 part2[RV / 2];
#pragma unroll
            for (int q = 0; q < RV / 2; ++q) part2[q] = 0ull;
            row_dot_pairs<RV, CW>(brow + i * S::BP + jc * CW, tpw + i * S::TPP + jc * S::PB, part2);
#pragma unroll
            for (int q = 0; q < RV / 2; ++q) add2(tot2[q], part2[q]);
          }
        }
#pragma unroll
        for (int q = 0; q < RV / 2; ++q) {  // raw numerators; the producers normalise
          out[2 * q + 1] = __uint_as_float((uint32_t)(tot2[q] & 0xFFFFFFFFull));
          out[2 * q] = __uint_as_float((uint32_t)(tot2[q] >> 32));
        }
      }
      mbar_arrive(&empty_b[s]);  // done reading stage s (pairs, regions, stats)
      if (tid == 0) PIV_STAMP(9, k);
      if (k >= 1) mbar_wait_bounded(&scempty_b, (uint32_t)((k - 1) & 1));
      if (tid == 0) PIV_STAMP(10, k);
      float* sc = Sc(wi) + row * S::SP + g * RV;
#pragma unroll
      for (int c = 0; c < RV; c += 4) *reinterpret_cast<float4*>(sc + c) = make_float4(out[c], out[c + 1], out[c + 2], out[c + 3]);
      mbar_arrive(&scfull_b);
    }
  }
}

// ================================================================== TM, tiny problems (one launch)
// For problems far below one wave (cfg 1: 64^2 frame, 16^2 template, 2,401 offsets) the step is
// launch- and latency-bound, so the whole path runs in ONE kernel: every CTA stages the template
// (prep a1: fp64 mean / energy, centred fp32 A_C, flat flag -- redundantly, a few hundred loads)
// and its band of image rows in shared memory; the window sums (a2) are fp64 column sums of h
// rows, then w of them per offset (exact for 2^-8-quantised inputs, any order); each thread takes
// offsets (u, v) and forms the numerator (a3: fp32, a fresh partial per template row, the order
// of tm_ncc_kernel's row-blocked partials), normalises (a4) and keys the argmax (a5); the frame's last CTA turns
// the key into its peak and resets the key / counter for the next call.
// grid = (ctas per frame, batch), block = 256; dynamic smem = 2 rows W doubles + (h w + (rows + h - 1) W)
// floats.
template <int TH, int TW>
__global__ void __launch_bounds__(256) tm_tiny_kernel(const float* __restrict__ img, int64_t pitch, int64_t frame_stride,
                                                      int W, const float* __restrict__ tmpl, int64_t tpitch, int h_rt,
                                                      int w_rt, int u_begin, int Ub, int V, int rows_per_cta,
                                                      float* __restrict__ scores, int64_t score_frame_stride,
                                                      unsigned long long* keys, unsigned int* done, PeakOut* peaks,
                                                      int ssd) {
  const int h = TH ? TH : h_rt, w = TW ? TW : w_rt, n = h * w;
  extern __shared__ double tiny_smd[];
  double* C1 = tiny_smd;                       // column sums over h rows: [rows][W] (fp64)
  double* C2 = C1 + (int64_t)rows_per_cta * W; // ... of squares
  float* T = reinterpret_cast<float*>(C2 + (int64_t)rows_per_cta * W);  // centred template, h x w
  float* X = T + n;                            // image rows [r0, r0 + rows + h - 1) of the band, W columns
  __shared__ double red[8];
  __shared__ unsigned long long redk[8];
  __shared__ bool last;
  const int f = blockIdx.y;
  const int r0 = blockIdx.x * rows_per_cta;
  const int rows = min(rows_per_cta, Ub - r0);
  // template: raw values, fp64 sum / sum of squares
  double s = 0.0, s2 = 0.0;
  for (int k = threadIdx.x; k < n; k += blockDim.x) {
    const float x = __ldg(tmpl + (int64_t)(k / w) * tpitch + k % w);
    T[k] = x;
    s += (double)x;
    s2 += (double)x * (double)x;
  }
  // image rows of this CTA
  const float* src = img + (int64_t)f * frame_stride + (int64_t)(u_begin + r0) * pitch;
  const int nr = rows + h - 1;
  {  // all of a thread's loads in flight before its stores (one memory round trip, not one per element)
    constexpr int LB = 8;
    const int ne = nr * W;
    for (int k0 = threadIdx.x; k0 < ne; k0 += LB * blockDim.x) {
      float v[LB];
#pragma unroll
      for (int r = 0; r < LB; ++r) {
        const int k = k0 + r * blockDim.x;
        v[r] = k < ne ? __ldg(src + (int64_t)(k / W) * pitch + k % W) : 0.0f;
      }
#pragma unroll
      for (int r = 0; r < LB; ++r) {
        const int k = k0 + r * blockDim.x;
        if (k < ne) X[k] = v[r];
      }
    }
  }
  s = block_sum_d(s, red);
  s2 = block_sum_d(s2, red);
  const double mean = s / (double)n, inv_n = 1.0 / (double)n;
  double e = 0.0, cs = 0.0;
  for (int k = threadIdx.x; k < n; k += blockDim.x) {
    const double a = (double)T[k] - mean;
    e += a * a;
    const float ac = (float)a;
    cs += (double)ac;
    T[k] = ac;  // each element is read and rewritten by the same thread
  }
  // window sums, separable: column sums of h rows, then (below) w of them per offset
  for (int k = threadIdx.x; k < rows * W; k += blockDim.x) {
    const int r = k / W, c = k % W;
    double a = 0.0, b = 0.0;
    for (int i = 0; i < h; ++i) {
      const double x = X[(r + i) * W + c];
      a += x;
      b = fma(x, x, b);
    }
    C1[k] = a;
    C2[k] = b;
  }
  e = block_sum_d(e, red);  // (its barriers also publish T, X, C1, C2)
  cs = block_sum_d(cs, red);
  const bool flat = e <= kFlatRel * s2;
  unsigned long long best = 0ull;
  for (int o = threadIdx.x; o < rows * V; o += blockDim.x) {
    const int ur = o / V, v = o % V;
    float num = 0.0f;
#pragma unroll 2
    for (int i = 0; i < h; ++i) {
      const float* xr = X + (ur + i) * W + v;
      const float* tr = T + i * w;
      float part = 0.0f;  // fresh partial per template row
#pragma unroll 8
      for (int j = 0; j < w; ++j) part = fmaf(tr[j], xr[j], part);
      num += part;
    }
    double s1 = 0.0, s2w = 0.0;
#pragma unroll 8
    for (int j = 0; j < w; ++j) {
      s1 += C1[ur * W + v + j];
      s2w += C2[ur * W + v + j];
    }
    const float sc = ssd ? (float)(s2 - 2.0 * ((double)num + mean * s1) + s2w)
                         : ncc_normalize_fast(num, s1, s2w, inv_n, cs, e, flat);
    const int u = u_begin + r0 + ur;
    if (scores) scores[(int64_t)f * score_frame_stride + (int64_t)(r0 + ur) * V + v] = sc;
    const unsigned long long key = make_key(ssd ? -sc : sc, (uint32_t)((int64_t)u * V + v));
    best = key > best ? key : best;
  }
  best = block_max_key(best, redk);
  if (threadIdx.x == 0) {
    if (best) atomicMax(keys + f, best);
    __threadfence();
    last = atomicAdd(done + f, 1u) == gridDim.x - 1;
  }
  __syncthreads();
  if (last && threadIdx.x == 0) {
    __threadfence();
    const unsigned long long k = atomicExch(keys + f, 0ull);  // read and reset for the next call
    const uint32_t idx = key_index(k);
    PeakOut pk;
    pk.score = ssd ? -key_score(k) : key_score(k);
    pk.u = (int32_t)(idx / (uint32_t)V);
    pk.v = (int32_t)(idx % (uint32_t)V);
    pk.flags = (flat && !ssd) ? (kFlatTemplate | kInvalid) : 0u;
    peaks[f] = pk;
    done[f] = 0u;
  }
}

}  // namespace nccb
