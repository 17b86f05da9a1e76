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
#include <cuda.h>  // CUtensorMap (type only; encoded on the host through the runtime entry point)
#include <cuda_runtime.h>
#include <stdint.h>

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
  int S;                     // split-K factor (fixed per variant: accumulation order depends on it)
};

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
  static constexpr int STAGE = ((T_BYTES + 127) / 128) * 128 + ((I_BYTES + 127) / 128) * 128;
  static constexpr int SMEM_TMA = 2 * STAGE;      // double-buffered (TMA path)
  static constexpr int SMEM_LDG = T_BYTES + I_BYTES;
  static_assert(IR <= 256 && IP <= 256 && CW <= 256 && CH <= 256, "TMA box dims are limited to 256");
};

// Numerator + fused normalise / clamp / optional surface store / CTA argmax (Fig 5.3-5.6).
// TH, TW: compile-time template size (specialised, "SK") or 0 (run-time evaluated, "RE").
// S: split of the (row-chunk, col-chunk) sequence of a tile over S CTAs; chunk ranges are fixed
//    per tile and the S partial totals are combined in index order by the last CTA to arrive, so
//    the result is deterministic and independent of scheduling and of the band (shard).
// TMA: stage image / template chunks with double-buffered cp.async.bulk.tensor + mbarrier;
//      otherwise (pitch not 16-B aligned) plain coalesced loads, single buffer.
// One CTA = one (tile, split) unit: blockIdx.x = tile * S + split, blockIdx.y = frame.
template <int RV, int LX, int WX, int WY, int CH, int CW, int TH, int TW, bool TMA>
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
  const int nCH = TH ? (TH + CH - 1) / CH : a.nCH;
  const int nCW = TW ? (TW + CW - 1) / CW : a.nCW;
  const int tplP = TW ? ((TW + CW - 1) / CW) * CW : a.tplP;

  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const int wx = wid % WX, wy = wid / WX;
  const int ly = lane / LX, lx = lane % LX;
  const int lu = wy * T::LY + ly;         // local output row
  const int lv = (wx * LX + lx) * RV;     // local output col (first of RV)
  const int f = blockIdx.y;
  const int S = a.S;
  const int tile = blockIdx.x / S, split = blockIdx.x % S;
  const int ty = tile / a.tiles_v, tx = tile % a.tiles_v;
  const int u0 = a.u_begin + ty * T::BU;
  const int v0 = tx * T::BV;
  const int nq = nCH * nCW;
  const int q0 = (split * nq) / S, q1 = ((split + 1) * nq) / S;  // this unit's chunk range

  float total[RV];
#pragma unroll
  for (int c = 0; c < RV; ++c) total[c] = 0.0f;

  auto compute_chunk = [&](const float* Ts, const float* Is) {
    const float* irow = Is + lu * T::IP + lv;
#pragma unroll 1
    for (int i = 0; i < CH; ++i) {
      float part[RV];
#pragma unroll
      for (int c = 0; c < RV; ++c) part[c] = 0.0f;
      row_dot<RV, CW>(irow + i * T::IP, Ts + i * CW, part);
#pragma unroll
      for (int c = 0; c < RV; ++c) total[c] += part[c];
    }
  };

  if constexpr (TMA) {
    auto stage_t = [&](int s) { return reinterpret_cast<float*>(smem_raw + s * T::STAGE); };
    auto stage_i = [&](int s) {
      return reinterpret_cast<float*>(smem_raw + s * T::STAGE + ((T::T_BYTES + 127) / 128) * 128);
    };
    auto issue = [&](int q, int s) {  // one thread: chunk q -> stage s
      const int ic = q / nCW, jc = q % nCW;
      mbar_expect_tx(&full_bar[s], (uint32_t)(T::T_BYTES + T::I_BYTES));
      tma_load_2d(stage_t(s), &map_tpl, jc * CW, ic * CH, &full_bar[s]);
      tma_load_3d(stage_i(s), &map_img, v0 + jc * CW, u0 + ic * CH, f, &full_bar[s]);
    };
    if (tid == 0) {
      tma_prefetch_desc(&map_img);
      tma_prefetch_desc(&map_tpl);
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
      compute_chunk(stage_t(s), stage_i(s));
      __syncthreads();  // every warp is done with stage s
      if (tid == 0 && q + 2 < q1) issue(q + 2, s);
    }
  } else {
    float* Ts = reinterpret_cast<float*>(smem_raw);
    float* Is = Ts + CH * CW;
    const float* img = a.img + (int64_t)f * a.frame_stride;
    for (int q = q0; q < q1; ++q) {
      const int ic = q / nCW, jc = q % nCW;
      __syncthreads();
      const float* tsrc = a.tplC + (int64_t)(ic * CH) * tplP + jc * CW;
      for (int k = tid; k < CH * CW; k += T::NT) Ts[k] = tsrc[(k / CW) * tplP + (k % CW)];
      const int gr0 = u0 + ic * CH, gc0 = v0 + jc * CW;
      for (int k = tid; k < T::IR * T::IP; k += T::NT) {
        const int r = k / T::IP, c = k % T::IP;
        const int gr = gr0 + r, gc = gc0 + c;
        Is[k] = (gr < a.H && gc < a.W) ? __ldg(img + (int64_t)gr * a.pitch + gc) : 0.0f;
      }
      __syncthreads();
      compute_chunk(Ts, Is);
    }
  }

  // ---- split-K combine: partials in fixed split order, by the last unit of the tile
  if (S > 1) {
    float* pbase = a.part + (((int64_t)f * a.tiles_u * a.tiles_v + tile) * S) * (RV * T::NT);
#pragma unroll
    for (int c = 0; c < RV; ++c) pbase[(int64_t)split * RV * T::NT + c * T::NT + tid] = total[c];
    __threadfence();
    __syncthreads();
    unsigned int* cnt = a.cnt + (int64_t)f * a.tiles_u * a.tiles_v + tile;
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
  const TemplateStats ts = *a.tst;
  const double n = (double)h * (double)w;
  const int u = u0 + lu;
  unsigned long long best = 0ull;
  if (u < a.u_end) {
    const int64_t rowoff = (int64_t)f * a.stat_frame_stride + (int64_t)(u - a.u_begin) * a.V;
    float* srow = a.scores ? a.scores + (int64_t)f * a.score_frame_stride + (int64_t)(u - a.u_begin) * a.V
                           : nullptr;
#pragma unroll
    for (int c = 0; c < RV; ++c) {
      const int v = v0 + lv + c;
      if (v < a.V) {
        const float sc = ncc_normalize(total[c], a.S1[rowoff + v], a.S2[rowoff + v], n, ts);
        if (srow) srow[v] = sc;
        const unsigned long long k = make_key(sc, (uint32_t)((int64_t)u * a.V + v));
        best = k > best ? k : best;
      }
    }
  }
  best = block_max_key(best, red_key);
  if (tid == 0 && best) atomicMax(a.keys + f, best);
}

// Template prep (Fig 5.2): Tbar, A_C = T - Tbar (fp32, zero-padded), A_D = sum A_C^2 (fp64),
// flat flag; resets the per-frame argmax keys.  One CTA, deterministic reductions.
__global__ void tm_template_prep(const float* __restrict__ tmpl, int64_t tpitch, int h, int w,
                                 float* __restrict__ tplC, int HP, int WP, TemplateStats* ts,
                                 unsigned long long* keys, int batch) {
  __shared__ double red[32];
  const int n = h * w;
  double s = 0.0, s2 = 0.0;
  for (int k = threadIdx.x; k < n; k += blockDim.x) {
    const double t = tmpl[(int64_t)(k / w) * tpitch + (k % w)];
    s += t;
    s2 += t * t;
  }
  s = block_sum_d(s, red);
  s2 = block_sum_d(s2, red);
  const double mean = s / (double)n;
  double e = 0.0, cs = 0.0;
  for (int k = threadIdx.x; k < HP * WP; k += blockDim.x) {
    const int i = k / WP, j = k % WP;
    float ac = 0.0f;
    if (i < h && j < w) {
      const double a = (double)tmpl[(int64_t)i * tpitch + j] - mean;
      e += a * a;
      ac = (float)a;
      cs += (double)ac;
    }
    tplC[k] = ac;
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
  for (int f = threadIdx.x; f < batch; f += blockDim.x) keys[f] = 0ull;
}

__global__ void tm_finalize(const unsigned long long* __restrict__ keys, const TemplateStats* ts, int V,
                            PeakOut* __restrict__ peaks, int batch) {
  const int f = blockIdx.x * blockDim.x + threadIdx.x;
  if (f >= batch) return;
  const unsigned long long k = keys[f];
  const uint32_t idx = key_index(k);
  PeakOut p;
  p.score = key_score(k);
  p.u = (int32_t)(idx / (uint32_t)V);
  p.v = (int32_t)(idx % (uint32_t)V);
  p.flags = ts->flat ? (kFlatTemplate | kInvalid) : 0u;
  peaks[f] = p;
}

// ================================================================== window sums (a2)
// Horizontal pass: RS[f][r][v] = sum_{j<w} I[row0 + r][v + j] for v < V (fp64), via a
// segment-local fp64 prefix sum staged in shared memory (exact for 2^-8-quantised inputs).
// grid = (ceil(V / SEG), rows, batch), block = NT.
template <int NT, int SEG>
__global__ void __launch_bounds__(NT)
    box_rows_kernel(const float* __restrict__ img, int64_t pitch, int64_t frame_stride, int W, int row0, int w,
                    int V, double* __restrict__ RS1, double* __restrict__ RS2, int64_t rs_frame_stride) {
  extern __shared__ double sm_d[];
  const int L = SEG + w;  // prefix entries P[0..L-1], P[k] = sum of the first k inputs
  double* P1 = sm_d;
  double* P2 = sm_d + L + 1;
  __shared__ double tot1[NT], tot2[NT];
  const int f = blockIdx.z, r = blockIdx.y;
  const int c0 = blockIdx.x * SEG;
  const float* src = img + (int64_t)f * frame_stride + (int64_t)(row0 + r) * pitch;
  const int cnt = min(L - 1, W - c0);  // inputs in this segment
  // per-thread contiguous block of inputs
  const int per = (L - 1 + NT - 1) / NT;
  const int b0 = threadIdx.x * per;
  double a1 = 0.0, a2 = 0.0;
  for (int k = 0; k < per; ++k) {
    const int idx = b0 + k;
    if (idx < cnt) {
      const double x = src[c0 + idx];
      a1 += x;
      a2 += x * x;
    }
  }
  tot1[threadIdx.x] = a1;
  tot2[threadIdx.x] = a2;
  __syncthreads();
  if (threadIdx.x == 0) {  // exclusive scan of the NT block totals (serial, deterministic)
    double s1 = 0.0, s2 = 0.0;
    for (int t = 0; t < NT; ++t) {
      const double q1 = tot1[t], q2 = tot2[t];
      tot1[t] = s1;
      tot2[t] = s2;
      s1 += q1;
      s2 += q2;
    }
  }
  __syncthreads();
  double s1 = tot1[threadIdx.x], s2 = tot2[threadIdx.x];
  if (threadIdx.x == 0) { P1[0] = 0.0; P2[0] = 0.0; }
  for (int k = 0; k < per; ++k) {
    const int idx = b0 + k;
    if (idx < L - 1) {
      const double x = idx < cnt ? (double)src[c0 + idx] : 0.0;
      s1 += x;
      s2 += x * x;
      P1[idx + 1] = s1;
      P2[idx + 1] = s2;
    }
  }
  __syncthreads();
  double* o1 = RS1 + (int64_t)f * rs_frame_stride + (int64_t)r * V;
  double* o2 = RS2 + (int64_t)f * rs_frame_stride + (int64_t)r * V;
  for (int k = threadIdx.x; k < SEG; k += NT) {
    const int v = c0 + k;
    if (v < V) {
      o1[v] = P1[k + w] - P1[k];
      o2[v] = P2[k + w] - P2[k];
    }
  }
}

// Vertical pass: S[f][u][v] = sum_{i<h} RS[f][u + i][v] for u < rows_out: direct sum for the
// first of RB rows, then sliding updates (fp64).  grid = (ceil(V/NT), ceil(rows_out/RB), batch).
template <int NT, int RB>
__global__ void __launch_bounds__(NT)
    box_cols_kernel(const double* __restrict__ RS1, const double* __restrict__ RS2, int64_t rs_frame_stride,
                    int V, int h, int rows_out, double* __restrict__ S1, double* __restrict__ S2,
                    int64_t s_frame_stride) {
  const int v = blockIdx.x * NT + threadIdx.x;
  if (v >= V) return;
  const int f = blockIdx.z;
  const int ub = blockIdx.y * RB;
  const double* r1 = RS1 + (int64_t)f * rs_frame_stride + v;
  const double* r2 = RS2 + (int64_t)f * rs_frame_stride + v;
  double* o1 = S1 + (int64_t)f * s_frame_stride + v;
  double* o2 = S2 + (int64_t)f * s_frame_stride + v;
  double a1 = 0.0, a2 = 0.0;
  for (int i = 0; i < h; ++i) {
    a1 += r1[(int64_t)(ub + i) * V];
    a2 += r2[(int64_t)(ub + i) * V];
  }
  const int ue = min(ub + RB, rows_out);
  for (int u = ub; u < ue; ++u) {
    if (u > ub) {
      a1 += r1[(int64_t)(u + h - 1) * V] - r1[(int64_t)(u - 1) * V];
      a2 += r2[(int64_t)(u + h - 1) * V] - r2[(int64_t)(u - 1) * V];
    }
    o1[(int64_t)u * V] = a1;
    o2[(int64_t)u * V] = a2;
  }
}

// ================================================================== PIV kernel (a6, a7)
struct PivArgs {
  const float* A;  // frames A (pairs), row pitch, frame stride in elements
  const float* B;
  int64_t pitch, frame_stride;
  int H, W, h, w, my, mx, sy, sx, Ky, Kx;
  const double* S1;  // window sums of frame B at every valid position: [pair][H-h+1][W-w+1]
  const double* S2;
  int64_t map_pitch, map_frame_stride;
  VecOut* vec;       // [pair][Ky][Kx]
  float* scores;     // nullable: [pair][Ky][Kx][OY][OX]
  int subpix;        // 0 Gauss3 (parabolic fallback), 1 parabola, 2 none
  int BP;            // RE: staged B pitch (floats), chosen on the host
};

template <int RV, int CW>
struct PivShape {
  int h, w, my, mx, OY, OX, NG, OXP, WP, BR, BP, items;
  __host__ __device__ PivShape(int h_, int w_, int my_, int mx_, int BP_)
      : h(h_), w(w_), my(my_), mx(mx_), OY(2 * my_ + 1), OX(2 * mx_ + 1), NG((2 * mx_ + 1 + RV - 1) / RV),
        OXP(((2 * mx_ + 1 + RV - 1) / RV) * RV), WP(((w_ + CW - 1) / CW) * CW), BR(h_ + 2 * my_), BP(BP_),
        items((2 * my_ + 1) * ((2 * mx_ + 1 + RV - 1) / RV)) {}
  __host__ __device__ int smem_floats() const { return h * WP + BR * BP + OY * OXP; }
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

// One CTA per (window k_x, window k_y, pair).  TH/TW/MY/MX: compile-time window and search
// sizes (SK) or 0 (RE).  CW = template columns per fp32 partial (and per unrolled row_dot).
template <int TH, int TW, int MY, int MX, int RV, int CW, int NT, int MINB>
__global__ void __launch_bounds__(NT, MINB) piv_ncc_kernel(const PivArgs a) {
  constexpr bool SK = TH > 0;
  const int BPc = SK ? piv_pick_pitch((((2 * MX + 1 + RV - 1) / RV) * RV) + (((TW + CW - 1) / CW) * CW), RV,
                                      (2 * MX + 1 + RV - 1) / RV)
                     : 0;
  const PivShape<RV, CW> sh(SK ? TH : a.h, SK ? TW : a.w, SK ? MY : a.my, SK ? MX : a.mx, SK ? BPc : a.BP);
  extern __shared__ float4 smem_f4[];
  float* As = reinterpret_cast<float*>(smem_f4);  // [h][WP]   mask A -> A_C
  float* Bs = As + sh.h * sh.WP;                  // [BR][BP]  search region of B
  float* Sc = Bs + sh.BR * sh.BP;                 // [OY][OXP] score tile
  __shared__ double red[32];
  __shared__ unsigned long long red_key[32];

  const int tid = threadIdx.x;
  const int kx = blockIdx.x, ky = blockIdx.y, pr = blockIdx.z;
  const int y = sh.my + ky * a.sy, x = sh.mx + kx * a.sx;
  const float* Af = a.A + (int64_t)pr * a.frame_stride;
  const float* Bf = a.B + (int64_t)pr * a.frame_stride;

  // ---- stage mask (zero-padded to WP) and search region (zero beyond the frame)
  for (int k = tid; k < sh.h * sh.WP; k += NT) {
    const int i = k / sh.WP, j = k % sh.WP;
    As[k] = j < sh.w ? __ldg(Af + (int64_t)(y + i) * a.pitch + (x + j)) : 0.0f;
  }
  const int by0 = y - sh.my, bx0 = x - sh.mx;
  for (int k = tid; k < sh.BR * sh.BP; k += NT) {
    const int i = k / sh.BP, j = k % sh.BP;
    const int gc = bx0 + j;
    Bs[k] = gc < a.W ? __ldg(Bf + (int64_t)(by0 + i) * a.pitch + gc) : 0.0f;
  }
  __syncthreads();

  // ---- mask statistics (Fig 5.2): mean, A_C in place, A_D, sum of fp32 A_C
  double s = 0.0, s2 = 0.0;
  for (int k = tid; k < sh.h * sh.WP; k += NT) {
    const double t = As[k];
    s += t;
    s2 += t * t;
  }
  s = block_sum_d(s, red);
  s2 = block_sum_d(s2, red);
  const double n = (double)sh.h * (double)sh.w;
  const double mean = s / n;
  double e = 0.0, cs = 0.0;
  for (int k = tid; k < sh.h * sh.WP; k += NT) {
    if (k % sh.WP < sh.w) {
      const double d = (double)As[k] - mean;
      e += d * d;
      const float ac = (float)d;
      cs += (double)ac;
      As[k] = ac;
    }
  }
  e = block_sum_d(e, red);  // contains __syncthreads: A_C visible afterwards
  cs = block_sum_d(cs, red);
  TemplateStats ts;
  ts.sum = s; ts.sumsq = s2; ts.energy = e; ts.csum = cs;
  ts.flat = (e <= kFlatRel * s2) ? 1 : 0;
  ts.pad = 0;

  // ---- numerator over flattened items (row, group of RV shifts) + normalisation
  const int nCW = sh.WP / CW;
  const double* S1f = a.S1 + (int64_t)pr * a.map_frame_stride;
  const double* S2f = a.S2 + (int64_t)pr * a.map_frame_stride;
  for (int it = tid; it < sh.items; it += NT) {
    const int row = it / sh.NG, g = it % sh.NG;
    float total[RV];
#pragma unroll
    for (int c = 0; c < RV; ++c) total[c] = 0.0f;
    const float* brow = Bs + row * sh.BP + g * RV;
#pragma unroll 1
    for (int i = 0; i < sh.h; ++i) {
#pragma unroll 1
      for (int jc = 0; jc < nCW; ++jc) {
        float part[RV];
#pragma unroll
        for (int c = 0; c < RV; ++c) part[c] = 0.0f;
        row_dot<RV, CW>(brow + i * sh.BP + jc * CW, As + i * sh.WP + jc * CW, part);
#pragma unroll
        for (int c = 0; c < RV; ++c) total[c] += part[c];
      }
    }
    const int64_t mrow = (int64_t)(y - sh.my + row) * a.map_pitch + (x - sh.mx);
#pragma unroll
    for (int c = 0; c < RV; ++c) {
      const int col = g * RV + c;
      float sc = 0.0f;
      if (col < sh.OX) sc = ncc_normalize(total[c], S1f[mrow + col], S2f[mrow + col], n, ts);
      Sc[row * sh.OXP + col] = sc;
    }
  }
  __syncthreads();

  // ---- argmax over the tile (tie -> smallest row-major index), optional surface store
  const int64_t wlin = ((int64_t)pr * a.Ky + ky) * a.Kx + kx;
  float* gsc = a.scores ? a.scores + wlin * sh.OY * sh.OX : nullptr;
  unsigned long long best = 0ull;
  for (int k = tid; k < sh.OY * sh.OX; k += NT) {
    const int row = k / sh.OX, col = k % sh.OX;
    const float sc = Sc[row * sh.OXP + col];
    if (gsc) gsc[k] = sc;
    const unsigned long long key = make_key(sc, (uint32_t)k);
    best = key > best ? key : best;
  }
  best = block_max_key(best, red_key);

  // ---- sub-pixel fit and the 24-B vector
  if (tid == 0) {
    const uint32_t k = key_index(best);
    const int row = (int)(k / sh.OX), col = (int)(k % sh.OX);
    const int iy = row - sh.my, ix = col - sh.mx;
    uint32_t flags = ts.flat ? (kFlatTemplate | kInvalid) : 0u;
    double ddy = 0.0, ddx = 0.0;
    bool par;
    if (row == 0 || row == sh.OY - 1) {
      flags |= kEdgeY;
    } else {
      ddy = subpix3(Sc[(row - 1) * sh.OXP + col], Sc[row * sh.OXP + col], Sc[(row + 1) * sh.OXP + col], a.subpix,
                    &par);
      if (par) flags |= kParabolaY;
    }
    if (col == 0 || col == sh.OX - 1) {
      flags |= kEdgeX;
    } else {
      ddx = subpix3(Sc[row * sh.OXP + col - 1], Sc[row * sh.OXP + col], Sc[row * sh.OXP + col + 1], a.subpix,
                    &par);
      if (par) flags |= kParabolaX;
    }
    VecOut o;
    o.iy = iy;
    o.ix = ix;
    o.dy = (float)(iy + ddy);
    o.dx = (float)(ix + ddx);
    o.score = key_score(best);
    o.flags = flags;
    a.vec[wlin] = o;
  }
}

}  // namespace nccb
