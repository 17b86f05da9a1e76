// ncc_piv_tc.cuh -- tensor-core (tcgen05, kind::f16, 3xBF16) numerator of the PIV path
// (SURVEY 8(f) row f3 extended to the batched PIV correlation of Figs 5.9-5.12).
//
// What it computes: for every interrogation window (mask T = frame A at (y, x), h x w) the
// numerator N[dy][dx] = sum_{i,j} A_C[i][j] * B[Y + dy + i][X + dx + j] over the search region
// of frame B (Y = y - m_y, X = x - m_x; dy in [0, 2 m_y], dx in [0, 2 m_x]), then the same
// normalisation, argmax and 3-point sub-pixel fit as the CUDA-core kernel (piv_ws2_kernel).
//
// Mapping onto the tensor cores (M = 128 accumulator lanes, K = template columns, N = output rows):
//   * R = 128 / D_x image rows per MMA (D_x = 2 m_x output columns per row: R = 2 at +-32,
//     R = 4 at +-16).  A lane m = D_x s + dx holds the Hankel row of image row r0 + s:
//     A[m][j] = B[r0 + s][X + dx + j], written by the producer warps into TMEM (tcgen05.st).
//   * The B operand is the REVERSED centred mask (K-major, rows 16 B apart, one zero row before
//     and 7 after it): the MMA of row group t (= r0 - Y) covers accumulator columns c in
//     [c_lo, c_lo + N) with B row n <-> template row i = t - c, so lane (s, dx), column c
//     accumulates A_C[i][.] . B[Y + t + s][X + dx + .] for output row dy = c + s.  Over the row
//     groups t = 0, R, 2R, ... column c of lane s collects exactly the template rows
//     i = -c (mod R); the R lanes of one dx cover the R residues: N[dy][dx] = sum_s D[D_x s + dx][dy - s]
//     (summed in s order by the drain warps).
//   * Adjacent windows of a column strip (same kx, ky = k0, k0 + 1, ...) overlap vertically: one
//     Hankel row group feeds the MMAs of every window whose search region contains it (up to
//     ceil((h + 2 m_y) / s_y) = 4 at cfg 3 / 4), each into its own accumulator slot (kNSlot
//     slots: the live windows + one being drained); the operand is built once per image row,
//     not once per window.
//   * 3xBF16 (kind::f16, K = 16 per MMA): x = hi + lo + r with hi = bf16(x), lo = bf16(x - hi),
//     |r| <= 2^-17 |x|; A.B ~ A_hi.B_hi + A_hi.B_lo + A_lo.B_hi (each bf16 product exact in the fp32
//     accumulator).  Per-product error ~2^-16 relative, random in sign: over the h w products of a
//     window ~2^-16 / sqrt(h w) of the normalisation (1e-7 at 64 x 64) -- and a bf16 MMA does K = 16
//     in the time a tf32 MMA does K = 8 (an M = 128 MMA takes max(45, N / 2) cycles either way,
//     tools/microbench/umma_probe.cu rates; this kernel's N is <= 80), so half the MMAs of 3xTF32.
//   * The last output column dx = 2 m_x (D_x + 1 columns do not fit R D_x = 128 lanes) comes from
//     a CUDA-core kernel (piv_tc_border_kernel) that runs before this one.
// Warp roles: 0-3 producers (Hankel operand -> TMEM, lane quadrant w), 4-7 drain / epilogue
// (accumulators -> shared surface, normalisation, argmax, sub-pixel), 8, 10, 11, 12 mask prep
// (statistics, centred hi/lo reversed operand), 9 TMA (search-region rows), 13-14 MMA issuers.
#pragma once
#include <cuda_bf16.h>
#include "ncc_tc.cuh"

namespace nccb {
namespace ptc {
constexpr int kNSlot = 5;   // accumulator + mask-operand slots (live windows + 1)
constexpr int kKs = 16;     // template columns per MMA K-step (bf16); a TMEM A chunk holds kc = 16 or 32
                            // of them (kc / 2 columns hi + kc / 2 lo: two bf16 per 32-bit column)
constexpr int kNAB = 3;     // TMEM A buffers (minimum; up to kNABMax when the accumulators leave room)
constexpr int kNABMax = 8;
constexpr int kNRing = 4;   // search-region row groups in flight (TMA)
constexpr int kNStat = 8;   // mask-statistics slots (prep -> epilogue), deeper than the operand slots
constexpr int kEpiWarp0 = 4, kTmaWarp = 9, kMmaWarp = 13, kNMma = 3;  // MMA warps 13 .. 12 + kNMma
// mask-prep warps 8, 10, 11, 12: none on the MMA warp's SMSP (warp % 4 == 1), whose issue slots
// the tensor pipe waits for; the TMA warp (nearly idle) takes warp 9
__host__ __device__ constexpr bool is_prep_warp(int w) { return w == 8 || w == 10 || w == 11 || w == 12; }
__host__ __device__ constexpr int prep_index(int w) { return w == 8 ? 0 : w - 9; }
constexpr int kThreads = (kMmaWarp + kNMma) * 32;
constexpr int kPrepMax = 32;  // mask elements per prep thread (h w <= 4096)
constexpr int kEpiB = 12, kEpiNB = 3, kEpiMax = kEpiB * kEpiNB;  // outputs per epilogue thread, in batches of kEpiB
__host__ __device__ constexpr int slot_cols(int my, int R) { return ((2 * my + R + 8) + 7) / 8 * 8; }
__host__ __device__ constexpr int b_rows(int h) { return h + 8; }  // 1 zero row + h + 7 zero rows
__host__ __device__ constexpr int b_slot_bytes(int h, int w) { return 2 * (w / 8) * b_rows(h) * 16; }  // bf16 hi + lo
__host__ __device__ constexpr int ring_pitch(int Dx, int w) { return ((Dx + w + 31) / 32) * 32; }  // floats (128 B rows)
__host__ __device__ constexpr int surf_pitch(int mx) { return ((2 * mx + 1) + 3) / 4 * 4; }
__host__ __device__ constexpr int smem_bytes(int h, int w, int my, int mx) {
  return kNSlot * b_slot_bytes(h, w) + kNRing * (128 / (2 * mx)) * ring_pitch(2 * mx, w) * 4 +
         (2 * my + 1) * surf_pitch(mx) * 4;
}
__host__ __device__ constexpr int chunk_cols(int w) { return w % 32 == 0 ? 32 : 16; }  // kc: TMEM columns = elements
__host__ __device__ constexpr int tmem_cols(int my, int R, int w) { return kNSlot * slot_cols(my, R) + kNAB * chunk_cols(w); }
// kind::f16 instruction descriptor: D f32, A/B bf16, both K-major, M = 128
__host__ __device__ constexpr uint32_t idesc_bf16(int N) {
  return (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);
}
__device__ __forceinline__ void mma_bf16_ts(uint32_t d, uint32_t a_tmem, uint64_t b, uint32_t idesc) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, 1, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n\t}" ::"r"(d),
      "r"(a_tmem), "l"(b), "r"(idesc)
      : "memory");
}
}  // namespace ptc

struct PivTcArgs {
  const float* A;         // frames A of the call (masks), absolute pair index
  int64_t pitch, frame_stride;
  int h, w, my, mx, sy, sx, Ky, Kx;
  int pair0;              // first pair of this launch (sub-batch)
  int R, Dx;              // image rows per MMA, output columns per image row (R Dx = 128)
  int nseg, segw, nunits; // column strips split into segments of segw windows; units of the launch
  const float *rsv, *mean;  // fp32 normalisation factors of frame B (box kernel), [z][map_h][map_w]
  int64_t map_pitch, map_frame_stride;
  const float* border;    // [z][Ky Kx][2 m_y + 1] numerators at dx = 2 m_x (piv_tc_border_kernel)
  VecOut* vec;            // [pair][Ky Kx]
  float* scores;          // nullable: [pair][Ky Kx][OY][OX]
  int subpix;
  unsigned long long* prof;  // nullable (NCC_PIV_TC_PROF): per-CTA wait accounting [grid][32] (globaltimer ns)
  int nab;  // TMEM A buffers (kNAB .. kNABMax: what the accumulator slots leave of the 512 columns)
  int exp;  // NCC_PIV_TC_EXP timing experiments (0 in normal use; results are wrong with bits set):
            // 1 producers skip the operand, 2 epilogue skips the normalisation, 4 prep skips the
            // mask work, 8 no MMAs
};

// Unit u of a launch: relative pair z, window column kx, windows ky in [k0, k0 + nw).
struct PivTcUnit {
  int z, kx, k0, nw;
};
__device__ __forceinline__ PivTcUnit piv_tc_unit(const PivTcArgs& a, int u) {
  PivTcUnit r;
  const int seg = u % a.nseg, rest = u / a.nseg;
  r.kx = rest % a.Kx;
  r.z = rest / a.Kx;
  r.k0 = seg * a.segw;
  r.nw = min(a.segw, a.Ky - r.k0);
  return r;
}

// grid = min(#SMs, nunits), block = ptc::kThreads, dynamic smem = ptc::smem_bytes(h, w, my, mx);
// map_b: frames B as (cols, rows, pair) fp32, box (D_x + w, 1, 1).
__global__ void __launch_bounds__(ptc::kThreads, 1) piv_tc_kernel(const PivTcArgs a,
                                                                  const __grid_constant__ CUtensorMap map_b) {
  using namespace ptc;
  extern __shared__ __align__(1024) unsigned char smem_pt[];
  __shared__ __align__(8) uint64_t img_full[kNRing], img_empty[kNRing], a_full[kNABMax], a_free[kNABMax],
      b_full[kNSlot], win_done[kNSlot], d_free[kNSlot], st_full[kNStat], epi_done[kNStat];
  __shared__ uint32_t tmem_base_s;
  __shared__ float st_csum[kNStat], st_rse[kNStat];
  __shared__ int st_flat[kNStat];
  __shared__ double red_s[8];
  __shared__ unsigned long long pkey_s[4];

  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int h = a.h, w = a.w, R = a.R, Dx = a.Dx;
  const int OY = 2 * a.my + 1, OX = 2 * a.mx + 1, OXP = surf_pitch(a.mx);
  const int SW = slot_cols(a.my, R), LB = b_rows(h), npl = w / 8, kc = chunk_cols(w), nkc = w / kc;
  const int bslot = b_slot_bytes(h, w);
  const int BPr = ring_pitch(Dx, w);
  const int span = h + 2 * a.my;  // search-region rows of one window
  const int nab = a.nab;           // TMEM A buffers
  const int nwin = a.Ky * a.Kx;
  float* ring = reinterpret_cast<float*>(smem_pt + kNSlot * bslot);
  float* P = ring + kNRing * R * BPr;

  // zero the mask operand slots (their pad rows stay zero) and the whole TMEM allocation
  {
    float4* z4 = reinterpret_cast<float4*>(smem_pt);
    for (int e = tid; e < kNSlot * bslot / 16; e += kThreads) z4[e] = make_float4(0.f, 0.f, 0.f, 0.f);
  }
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_u32(&tmem_base_s)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (tid == 0) {
    for (int b = 0; b < kNRing; ++b) {
      mbar_init(&img_full[b], 1);
      mbar_init(&img_empty[b], 128);
    }
    for (int b = 0; b < kNABMax; ++b) {
      mbar_init(&a_full[b], 128);
      mbar_init(&a_free[b], kNMma);  // one commit per MMA warp
    }
    for (int b = 0; b < kNSlot; ++b) {
      mbar_init(&b_full[b], 128);
      mbar_init(&win_done[b], 1);
      mbar_init(&d_free[b], 128);
    }
    for (int b = 0; b < kNStat; ++b) {
      mbar_init(&st_full[b], 1);
      mbar_init(&epi_done[b], 1);
    }
    fence_mbar_init();
  }
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const uint32_t tbase = tmem_base_s;
  const uint32_t acol0 = (uint32_t)(kNSlot * SW);  // A buffers after the accumulator slots
  // NCC_PIV_TC_PROF: one thread per role accumulates its waits (SM clock cycles), added to
  // prof[cta][slot] at the end (tools/piv_tc_prof.py)
  unsigned long long* const prof = a.prof;
  auto pclock = []() { return (unsigned long long)clock64(); };
  unsigned long long pacc[6] = {0ull, 0ull, 0ull, 0ull, 0ull, 0ull};
  const unsigned long long pt_start = prof ? pclock() : 0ull;
  auto twait = [&](uint64_t* bar, uint32_t par, int k) {
    if (prof) {
      const unsigned long long t0 = pclock();
      mbar_wait_bounded(bar, par);
      pacc[k] += pclock() - t0;
    } else {
      mbar_wait_bounded(bar, par);
    }
  };
  auto pflush = [&](int base, bool me) {
    if (prof && me) {
      atomicAdd(prof + blockIdx.x * 32 + base, pclock() - pt_start);
#pragma unroll
      for (int k = 0; k < 6; ++k) atomicAdd(prof + blockIdx.x * 32 + base + 1 + k, pacc[k]);
    }
  };
  if (warp < 4) {
    const uint32_t z[8] = {0u, 0u, 0u, 0u, 0u, 0u, 0u, 0u};
    const uint32_t lb = (uint32_t)(warp * 32) << 16;
    for (int c = 0; c < 512; c += 8) tc::st8(tbase + lb + (uint32_t)c, z);
    tc::st_wait();
  }
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  tc::fence_before();
  __syncthreads();
  tc::fence_after();

  if (warp < 4) {
    // ===================== producers: lane m = D_x s + dx -> Hankel row of image row r0 + s (a warp
    // reads consecutive columns of one staged row: conflict-free)
    const int m = warp * 32 + lane, s = m / Dx, dx = m % Dx;
    const uint32_t lane_base = (uint32_t)(warp * 32) << 16;
    int gq = 0, cq = 0, b = 0, ph = 0;
    for (int u = blockIdx.x; u < a.nunits; u += gridDim.x) {
      const PivTcUnit un = piv_tc_unit(a, u);
      const int ng = ((un.nw - 1) * a.sy + span + R - 1) / R;
      for (int g = 0; g < ng; ++g, ++gq) {
        const int rs = gq & (kNRing - 1);
        twait(&img_full[rs], (uint32_t)((gq / kNRing) & 1), 0);
        const float* row0 = ring + (rs * R + s) * BPr + (dx & ~1);
        const bool odd = (dx & 1) != 0;
        for (int q = 0; q < nkc; ++q, ++cq) {
          // kc elements -> kc / 2 columns of (bf16 hi) pairs and kc / 2 of (bf16 lo) pairs, the even
          // element in the low half of each 32-bit cell
          // 8-byte loads from the even column at or below dx + j (lanes 2i and 2i+1 share them),
          // odd lanes take the pair shifted by one; packed conversions (cvt.rn.bf16x2.f32)
          uint32_t hi[16], lo[16];
          const float2* r2 = reinterpret_cast<const float2*>(row0 + q * kc);
          float2 cur = (a.exp & 1) ? make_float2(0.f, 0.f) : r2[0];
#pragma unroll
          for (int p = 0; p < 16; ++p) {
            if (2 * p < kc) {
              const float2 nxt = (a.exp & 1) ? make_float2(0.f, 0.f) : r2[p + 1];
              const float x0 = odd ? cur.y : cur.x, x1 = odd ? nxt.x : cur.y;
              cur = nxt;
              const __nv_bfloat162 hv = __floats2bfloat162_rn(x0, x1);
              const uint32_t hu = *reinterpret_cast<const uint32_t*>(&hv);
              const __nv_bfloat162 lv =
                  __floats2bfloat162_rn(x0 - __uint_as_float(hu << 16), x1 - __uint_as_float(hu & 0xffff0000u));
              hi[p] = hu;
              lo[p] = *reinterpret_cast<const uint32_t*>(&lv);
            }
          }
          if (cq >= nab) {  // the buffer's previous chunk (one round back) consumed
            twait(&a_free[b], (uint32_t)(ph ^ 1), 1);
            tc::fence_after();
          }
          const uint32_t ab = tbase + lane_base + acol0 + (uint32_t)(b * kc);
          if (!(a.exp & 1)) {
            tc::st8(ab, *reinterpret_cast<const uint32_t(*)[8]>(hi));
            tc::st8(ab + kc / 2, *reinterpret_cast<const uint32_t(*)[8]>(lo));
            if (kc == 32) {
              tc::st8(ab + 8, *reinterpret_cast<const uint32_t(*)[8]>(hi + 8));
              tc::st8(ab + 24, *reinterpret_cast<const uint32_t(*)[8]>(lo + 8));
            }
          }
          tc::st_wait();
          tc::fence_before();
          mbar_arrive(&a_full[b]);
          if (++b == nab) {
            b = 0;
            ph ^= 1;
          }
        }
        mbar_arrive(&img_empty[rs]);
      }
    }
  } else if (warp == kTmaWarp) {
    // ===================== TMA: R search-region rows per group, kNRing groups ahead
    if (lane == 0) {
      tma_prefetch_desc(&map_b);
      int gq = 0;
      for (int u = blockIdx.x; u < a.nunits; u += gridDim.x) {
        const PivTcUnit un = piv_tc_unit(a, u);
        const int ng = ((un.nw - 1) * a.sy + span + R - 1) / R;
        const int X = un.kx * a.sx, Y0 = un.k0 * a.sy;
        for (int g = 0; g < ng; ++g, ++gq) {
          const int rs = gq % kNRing;
          if (gq >= kNRing) mbar_wait_bounded(&img_empty[rs], (uint32_t)(((gq / kNRing) - 1) & 1));
          mbar_expect_tx(&img_full[rs], (uint32_t)(R * (Dx + w) * 4));
          for (int s = 0; s < R; ++s)
            tma_load_3d(ring + (rs * R + s) * BPr, &map_b, X, Y0 + R * g + s, a.pair0 + un.z, &img_full[rs]);
        }
      }
    }
    __syncwarp();
  } else if (is_prep_warp(warp)) {
    // ===================== mask prep: statistics (Fig 5.2) and the reversed centred hi/lo operand
    const int pw = prep_index(warp), pt = pw * 32 + lane;
    const int ne = (a.exp & 4) ? 0 : h * w / 128;  // elements per thread (element pt + 128 k)
    const double inv_n = 1.0 / ((double)h * (double)w);
    int wseq = 0;
    auto reduce2 = [&](double& x0, double& x1) {  // deterministic sums over the 128 prep threads
      x0 = warp_sum_d(x0);
      x1 = warp_sum_d(x1);
      named_bar_sync(2, 128);
      if (lane == 0) {
        red_s[2 * pw] = x0;
        red_s[2 * pw + 1] = x1;
      }
      named_bar_sync(2, 128);
      x0 = (red_s[0] + red_s[2]) + (red_s[4] + red_s[6]);
      x1 = (red_s[1] + red_s[3]) + (red_s[5] + red_s[7]);
      named_bar_sync(2, 128);
    };
    for (int u = blockIdx.x; u < a.nunits; u += gridDim.x) {
      const PivTcUnit un = piv_tc_unit(a, u);
      for (int i = 0; i < un.nw; ++i, ++wseq) {
        const int sl = wseq % kNSlot, use = wseq / kNSlot;
        const int ky = un.k0 + i;
        const float* Aw = a.A + (int64_t)(a.pair0 + un.z) * a.frame_stride +
                          (int64_t)(a.my + ky * a.sy) * a.pitch + (a.mx + un.kx * a.sx);
        float v[kPrepMax];
        double s1 = 0.0, s2 = 0.0;
#pragma unroll
        for (int k = 0; k < kPrepMax; ++k) {
          if (k < ne) {
            const int e = pt + 128 * k;
            v[k] = __ldg(Aw + (int64_t)(e / w) * a.pitch + e % w);
            s1 += (double)v[k];
            s2 += (double)v[k] * (double)v[k];
          }
        }
        reduce2(s1, s2);
        const double mean = s1 * inv_n, sumsq = s2;
        // operand slot: the MMAs of its previous window complete; statistics slot: the epilogue
        // of its previous window (kNStat windows back) done
        const int st = wseq % kNStat, su = wseq / kNStat;
        if (use >= 1) twait(&win_done[sl], (uint32_t)((use - 1) & 1), 0);
        if (su >= 1) twait(&epi_done[st], (uint32_t)((su - 1) & 1), 1);
        uint16_t* bh = reinterpret_cast<uint16_t*>(smem_pt + sl * bslot);
        uint16_t* bl = bh + npl * LB * 8;
        double en = 0.0, cs = 0.0;
#pragma unroll
        for (int k = 0; k < kPrepMax; ++k) {
          if (k < ne) {
            const int e = pt + 128 * k, ii = e / w, j = e % w;
            const double d = (double)v[k] - mean;
            const float ac = (float)d;
            en += d * d;
            cs += (double)ac;
            const __nv_bfloat16 hb = __float2bfloat16_rn(ac);
            const int off = ((j >> 3) * LB + (h - ii)) * 8 + (j & 7);  // row q = h - 1 - i, +1 pre-pad row
            bh[off] = __bfloat16_as_ushort(hb);
            bl[off] = __bfloat16_as_ushort(__float2bfloat16_rn(ac - __bfloat162float(hb)));
          }
        }
        reduce2(en, cs);
        if (pt == 0) {
          const bool flat = en <= kFlatRel * sumsq;
          st_flat[st] = flat ? 1 : 0;
          st_csum[st] = (float)cs;
          st_rse[st] = flat ? 0.0f : (float)(1.0 / sqrt(en));
          mbar_arrive(&st_full[st]);
        }
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // operand visible to the tensor core
        mbar_arrive(&b_full[sl]);
      }
    }
  } else if (warp >= kEpiWarp0 && warp < kEpiWarp0 + 4) {
    // ===================== drain + epilogue: lane m = D_x s + dx reads accumulator lane m
    const int et = tid - kEpiWarp0 * 32, wq = warp & 3;
    const int m = wq * 32 + lane, s = m / Dx, dx = m % Dx;
    const uint32_t lane_base = (uint32_t)(wq * 32) << 16;
    const uint32_t z[8] = {0u, 0u, 0u, 0u, 0u, 0u, 0u, 0u};
    const int tile = OY * OX;
    const int e_dy = 128 / OX, e_dx = 128 % OX;  // output e -> e + 128: (row, column) steps
    const int ey0 = et / OX, ex0 = et % OX;      // first output of this thread
    int wseq = 0;
    for (int u = blockIdx.x; u < a.nunits; u += gridDim.x) {
      const PivTcUnit un = piv_tc_unit(a, u);
      for (int i = 0; i < un.nw; ++i, ++wseq) {
        const int sl = wseq % kNSlot, use = wseq / kNSlot;
        const int ky = un.k0 + i, lin = ky * a.Kx + un.kx;
        // the window's normalisation factors do not depend on its accumulators: the first batch of
        // this thread's outputs (e = et + 128 c) is requested before the wait and lands during it,
        // each later batch after the previous one is normalised
        const int64_t mo = (int64_t)un.z * a.map_frame_stride + (int64_t)(ky * a.sy) * a.map_pitch + un.kx * a.sx;
        float fr[kEpiB], fm[kEpiB];
        auto load_batch = [&](int ey, int ex) {
#pragma unroll
          for (int c = 0; c < kEpiB; ++c) {
            if (ey < OY) {
              const int64_t mi = mo + (int64_t)ey * a.map_pitch + ex;
              fr[c] = __ldg(a.rsv + mi);
              fm[c] = __ldg(a.mean + mi);
            }
            ex += e_dx;
            ey += e_dy;
            if (ex >= OX) {
              ex -= OX;
              ++ey;
            }
          }
        };
        load_batch(ey0, ex0);
        const int st = wseq % kNStat, su = wseq / kNStat;
        twait(&win_done[sl], (uint32_t)(use & 1), 0);
        tc::fence_after();
        const unsigned long long t_dr = prof ? pclock() : 0ull;
        const uint32_t sbase = tbase + lane_base + (uint32_t)(sl * SW);
        // N[dy][dx] = sum_s D[D_x s + dx][dy - s + R] (slot column index = c + R), in s order: the
        // warps of sub-row s (lane quadrants) store / add in pass s
        for (int pass = 0; pass < R; ++pass) {
          if (s == pass) {
            for (int cc = 0; cc < SW; cc += 8) {
              uint32_t d[8];
              tc::ld8(sbase + (uint32_t)cc, d);
#pragma unroll
              for (int e = 0; e < 8; ++e) {
                const int dy = cc + e - R + s;
                if (dy >= 0 && dy < OY) {
                  float* pp = P + dy * OXP + dx;
                  *pp = pass == 0 ? __uint_as_float(d[e]) : *pp + __uint_as_float(d[e]);
                }
              }
            }
          }
          named_bar_sync(3, 128);
        }
        for (int cc = 0; cc < SW; cc += 8) tc::st8(sbase + (uint32_t)cc, z);
        tc::st_wait();
        tc::fence_before();
        mbar_arrive(&d_free[sl]);
        if (prof) pacc[1] += pclock() - t_dr;
        twait(&st_full[st], (uint32_t)(su & 1), 2);  // the window's mask statistics
        if (a.exp & 2) {
          if (et == 0) mbar_arrive(&epi_done[st]);
          continue;
        }
        const float* bd = a.border + ((int64_t)un.z * nwin + lin) * OY;
        for (int dy = et; dy < OY; dy += 128) P[dy * OXP + Dx] = __ldg(bd + dy);
        named_bar_sync(3, 128);
        // normalise (fp32 factors of the window kernel, as piv_ws2_kernel), argmax keys
        const float csf = st_csum[st], rse = st_rse[st];
        float* gsc = a.scores ? a.scores + ((int64_t)(a.pair0 + un.z) * nwin + lin) * tile : nullptr;
        unsigned long long best = 0ull;
        auto norm_batch = [&](int ey, int ex) {
#pragma unroll
          for (int c = 0; c < kEpiB; ++c) {
            if (ey < OY) {
              float* tp = P + ey * OXP + ex;
              const float r0 = fmaf(-csf, fm[c], *tp) * (fr[c] * rse);
              const float sv = r0 > 1.0f ? 1.0f : (r0 < -1.0f ? -1.0f : r0);
              *tp = sv;
              const int e = ey * OX + ex;
              if (gsc) gsc[e] = sv;
              const unsigned long long key = make_key(sv, (uint32_t)e);
              best = key > best ? key : best;
            }
            ex += e_dx;
            ey += e_dy;
            if (ex >= OX) {
              ex -= OX;
              ++ey;
            }
          }
        };
        norm_batch(ey0, ex0);
        for (int bt = 1; bt < kEpiNB; ++bt) {
          const int eb = et + 128 * kEpiB * bt;
          if (eb >= tile) break;
          load_batch(eb / OX, eb % OX);
          norm_batch(eb / OX, eb % OX);
        }
        best = warp_max_key(best);
        if (lane == 0) pkey_s[wq] = best;
        named_bar_sync(3, 128);
        if (et == 0) {
          unsigned long long bk = pkey_s[0];
          for (int q = 1; q < 4; ++q) bk = pkey_s[q] > bk ? pkey_s[q] : bk;
          const uint32_t kk = key_index(bk);
          const int row = (int)(kk / OX), col = (int)(kk % OX);
          const int iy = row - a.my, ix = col - a.mx;
          uint32_t flags = st_flat[st] ? (kFlatTemplate | kInvalid) : 0u;
          double ddy = 0.0, ddx = 0.0;
          bool par = false;
          if (row == 0 || row == OY - 1) {
            flags |= kEdgeY;
          } else {
            ddy = subpix3(P[(row - 1) * OXP + col], P[row * OXP + col], P[(row + 1) * OXP + col], a.subpix, &par);
            if (par) flags |= kParabolaY;
          }
          par = false;
          if (col == 0 || col == OX - 1) {
            flags |= kEdgeX;
          } else {
            ddx = subpix3(P[row * OXP + col - 1], P[row * OXP + col], P[row * OXP + col + 1], a.subpix, &par);
            if (par) flags |= kParabolaX;
          }
          VecOut o;
          o.iy = iy;
          o.ix = ix;
          o.dy = (float)(iy + ddy);
          o.dx = (float)(ix + ddx);
          o.score = key_score(bk);
          o.flags = flags;
          a.vec[(int64_t)(a.pair0 + un.z) * nwin + lin] = o;
        }
        named_bar_sync(3, 128);  // surface read; the slot's statistics may be replaced
        if (et == 0) mbar_arrive(&epi_done[st]);
      }
    }
  } else if (warp >= kMmaWarp) {
    // ===================== MMA issuer.  The whole warp walks the schedule (warp-uniform values
    // stay in uniform registers), one elected lane issues.  Per row group each live window's
    // operands follow from its row offset t = R k alone (a few integer operations); per K chunk
    // only a constant is added.
    const int KT = (span + R - 1) / R;  // row groups per window
    const bool leader = tc::elect_one();
    const uint32_t bsm = smem_u32(smem_pt);
    const uint32_t plane = (uint32_t)LB * 16;
    const uint64_t dconst = tc::sdesc(0u, plane, 128);
    const uint64_t lo_off = (uint64_t)(((uint32_t)npl * LB * 16) >> 4);  // hi -> lo operand (descriptor units)
    const uint64_t kstep = (uint64_t)((2u * plane) >> 4);                 // one K-step of 16 = two planes of 8
    const uint64_t qstep = (uint64_t)(((uint32_t)(kc / 8) * plane) >> 4);   // one K chunk
    const int gpw = a.sy / R;  // row groups between two window starts
    // kNMma issuing warps share the live windows by sequence parity: every accumulator is written
    // by one warp only, in its fixed order (deterministic); each warp releases the A buffers
    const int mpar = warp - kMmaWarp;
    int b = 0, ph = 0, wseq = 0, ntr = 0;
    for (int u = blockIdx.x; u < a.nunits; u += gridDim.x) {
      const PivTcUnit un = piv_tc_unit(a, u);
      const int ng = ((un.nw - 1) * a.sy + span + R - 1) / R;
      // live windows, oldest first: slot, slot use, accumulator base, operand base, first group
      int wsl[kNSlot - 1], wuse[kNSlot - 1], wg0[kNSlot - 1];
      bool wmine[kNSlot - 1];
      uint32_t wdb[kNSlot - 1], wbb[kNSlot - 1];
#pragma unroll
      for (int li = 0; li < kNSlot - 1; ++li) {
        wsl[li] = wuse[li] = wg0[li] = 0;
        wmine[li] = false;
        wdb[li] = wbb[li] = 0u;
      }
      int nlive = 0, inext = 0;
      for (int g = 0; g < ng; ++g) {
        if (inext < un.nw && g == inext * gpw) {  // a window starts at this row group
#pragma unroll
          for (int li = 0; li < kNSlot - 1; ++li)
            if (li == nlive) {
              const int sl = wseq % kNSlot;
              wsl[li] = sl;
              wuse[li] = wseq / kNSlot;
              wmine[li] = (wseq % kNMma) == mpar;
              wg0[li] = g;
              wdb[li] = tbase + (uint32_t)(sl * SW);
              wbb[li] = bsm + (uint32_t)(sl * bslot);
            }
          ++nlive;
          ++inext;
          ++wseq;
        }
        uint32_t dcol[kNSlot - 1], idd[kNSlot - 1];
        uint64_t dh0[kNSlot - 1];
#pragma unroll
        for (int li = 0; li < kNSlot - 1; ++li) {
          const int t = R * (g - wg0[li]);
          const int c_a = max(-(R - 1), t - h + 1), c_b = min(2 * a.my, t);
          const int c_lo = c_a - ((c_a + R) & 1);  // even accumulator column
          const int N = ((c_b - c_lo + 1) + 7) & ~7;
          dcol[li] = wdb[li] + (uint32_t)(c_lo + R);
          idd[li] = idesc_bf16(N);
          // B row of column c_lo: template row t - c_lo (+1 pre-pad row)
          dh0[li] = dconst + (uint64_t)((wbb[li] + (uint32_t)(h - t + c_lo) * 16u) >> 4);
        }
        uint64_t qoff = 0;
        for (int q = 0; q < nkc; ++q, qoff += qstep) {
          const unsigned long long tw = prof ? pclock() : 0ull;
          twait(&a_full[b], (uint32_t)ph, 0);
          const unsigned long long tq = prof ? pclock() : 0ull;
          tc::fence_after();
          const uint32_t ah0 = tbase + acol0 + (uint32_t)(b * kc);
#pragma unroll
          for (int li = 0; li < kNSlot - 1; ++li) {
            if (li >= nlive || !wmine[li]) continue;
            if (q == 0 && g == wg0[li]) {  // the window's first MMA: operand prepared, accumulator slot drained
              twait(&b_full[wsl[li]], (uint32_t)(wuse[li] & 1), 1);
              if (wuse[li] >= 1) twait(&d_free[wsl[li]], (uint32_t)((wuse[li] - 1) & 1), 2);
              tc::fence_after();
            }
            if (leader && !(a.exp & 8)) {
              uint64_t dh = dh0[li] + qoff;
#pragma unroll
              for (int kk = 0; kk < kc / kKs; ++kk, dh += kstep) {
                const uint32_t ah = ah0 + (uint32_t)(kk * 8);
                mma_bf16_ts(dcol[li], ah, dh, idd[li]);
                mma_bf16_ts(dcol[li], ah, dh + lo_off, idd[li]);
                mma_bf16_ts(dcol[li], ah + kc / 2, dh, idd[li]);
              }
            }
          }
          if (leader) {
            tc::commit(&a_free[b]);
            if (q == nkc - 1 && nlive > 0 && wmine[0] && g - wg0[0] == KT - 1) tc::commit(&win_done[wsl[0]]);
          }
          __syncwarp();
          if (prof) {
            const unsigned long long te = pclock();
            pacc[3] += te - tq;
            if (blockIdx.x == 0 && lane == 0 && warp == kMmaWarp && ntr < 2048) {  // trace of CTA 0's first chunks
              prof[gridDim.x * 32 + 3 * ntr] = tw;
              prof[gridDim.x * 32 + 3 * ntr + 1] = tq;
              prof[gridDim.x * 32 + 3 * ntr + 2] = te;
            }
            ++ntr;
          }
          if (++b == nab) {
            b = 0;
            ph ^= 1;
          }
        }
        if (nlive > 0 && g - wg0[0] == KT - 1) {  // the oldest window is complete: retire it
#pragma unroll
          for (int li = 0; li < kNSlot - 2; ++li) {
            wsl[li] = wsl[li + 1];
            wuse[li] = wuse[li + 1];
            wmine[li] = wmine[li + 1];
            wg0[li] = wg0[li + 1];
            wdb[li] = wdb[li + 1];
            wbb[li] = wbb[li + 1];
          }
          --nlive;
        }
      }
    }
  }
  if (warp < 4) pflush(0, tid == 0);
  else if (is_prep_warp(warp)) pflush(8, warp == 8 && lane == 0);
  else if (warp >= kEpiWarp0 && warp < kEpiWarp0 + 4) pflush(16, tid == kEpiWarp0 * 32);
  else if (warp == kMmaWarp) pflush(24, lane == 0);
  tc::fence_before();
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tbase));
}

// The last output column dx = 2 m_x of every window on the CUDA cores (the tensor-core kernel
// covers dx < 2 m_x): N[dy][2 m_x] = sum_{i,j} A_C[i][j] B[Y + dy + i][X + 2 m_x + j], A_C from
// the fp64 mean of the mask.  grid = (Ky Kx, pairs of the launch), block = 256: warp wp takes the
// output rows dy = 9 wp .. 9 wp + 8, lane the template columns j = lane + 32 c; per template row a
// sliding register window of the 9 image rows it meets, then one butterfly sum per output.
// dynamic smem = (h w + (h + 2 m_y + 8) w) floats.
constexpr int kBorderDY = 9;
__global__ void __launch_bounds__(256) piv_tc_border_kernel(const PivTcArgs a, const float* __restrict__ Bf) {
  extern __shared__ __align__(16) float sm_bd[];
  __shared__ double red[8];
  const int h = a.h, w = a.w, OY = 2 * a.my + 1, span = h + 2 * a.my;
  float* T = sm_bd;
  float* Bc = sm_bd + h * w;
  const int lin = blockIdx.x, z = blockIdx.y;
  const int ky = lin / a.Kx, kx = lin % a.Kx;
  const int y = a.my + ky * a.sy, x = a.mx + kx * a.sx;
  const float* Aw = a.A + (int64_t)(a.pair0 + z) * a.frame_stride + (int64_t)y * a.pitch + x;
  const float* Bw = Bf + (int64_t)(a.pair0 + z) * a.frame_stride + (int64_t)(y - a.my) * a.pitch + x + a.mx;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  double s1 = 0.0;
  // staging: one row per warp pass, lanes along the row (no per-element division)
  for (int i = warp; i < h; i += 8)
    for (int j = lane; j < w; j += 32) {
      const float v = __ldg(Aw + (int64_t)i * a.pitch + j);
      T[i * w + j] = v;
      s1 += (double)v;
    }
  for (int i = warp; i < span + kBorderDY - 1; i += 8)
    for (int j = lane; j < w; j += 32) Bc[i * w + j] = i < span ? __ldg(Bw + (int64_t)i * a.pitch + j) : 0.0f;
  s1 = warp_sum_d(s1);
  if (lane == 0) red[warp] = s1;
  __syncthreads();
  double tot = 0.0;
  for (int q = 0; q < 8; ++q) tot += red[q];
  const double mean = tot / ((double)h * (double)w);
  for (int i = warp; i < h; i += 8)
    for (int j = lane; j < w; j += 32) T[i * w + j] = (float)((double)T[i * w + j] - mean);
  __syncthreads();
  const int dy0 = warp * kBorderDY;
  if (dy0 >= OY) return;
  float acc[kBorderDY];
#pragma unroll
  for (int d = 0; d < kBorderDY; ++d) acc[d] = 0.0f;
  for (int j = lane; j < w; j += 32) {
    float xw[kBorderDY];
#pragma unroll
    for (int d = 0; d < kBorderDY - 1; ++d) xw[d + 1] = Bc[(dy0 + d) * w + j];
    for (int i = 0; i < h; ++i) {
#pragma unroll
      for (int d = 0; d < kBorderDY - 1; ++d) xw[d] = xw[d + 1];
      xw[kBorderDY - 1] = Bc[(dy0 + i + kBorderDY - 1) * w + j];
      const float t = T[i * w + j];
#pragma unroll
      for (int d = 0; d < kBorderDY; ++d) acc[d] = fmaf(t, xw[d], acc[d]);
    }
  }
#pragma unroll
  for (int d = 0; d < kBorderDY; ++d) {
    float v = acc[d];
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    if (lane == 0 && dy0 + d < OY) const_cast<float*>(a.border)[((int64_t)z * a.Ky * a.Kx + lin) * OY + dy0 + d] = v;
  }
}


// Register-blocked form for TH = h in {32, 64} and w a multiple of 32: warp (b, c) takes the 9
// output rows dy = 9 b + d and the template columns j = 32 c + lane; each thread keeps its
// template column in registers and streams the image column once (row r' of the block meets
// template rows r' - d: compile-time after unrolling), ~9 FMAs per shared load.  grid = (Ky Kx,
// pairs), block = 8 (w / 32) warps; dynamic smem as piv_tc_border_kernel + 8 (w / 32) 9 floats.
template <int TH>
__global__ void __launch_bounds__(512) piv_tc_border_rb(const PivTcArgs a, const float* __restrict__ Bf) {
  extern __shared__ __align__(16) float sm_rb[];
  __shared__ double red[16];
  const int w = a.w, OY = 2 * a.my + 1, span = TH + 2 * a.my, ncw = w / 32, nth = 256 * ncw;
  float* T = sm_rb;
  float* Bc = sm_rb + TH * w;
  float* part = Bc + (span + kBorderDY - 1) * w;  // [ncw][8][9]
  const int lin = blockIdx.x, z = blockIdx.y;
  const int ky = lin / a.Kx, kx = lin % a.Kx;
  const int y = a.my + ky * a.sy, x = a.mx + kx * a.sx;
  const float* Aw = a.A + (int64_t)(a.pair0 + z) * a.frame_stride + (int64_t)y * a.pitch + x;
  const float* Bw = Bf + (int64_t)(a.pair0 + z) * a.frame_stride + (int64_t)(y - a.my) * a.pitch + x + a.mx;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5, nwarp = nth / 32;
  double s1 = 0.0;
  // The CTA is load-latency bound (one window's 64-wide strips, ~51 KB): with 16-byte aligned rows
  // every thread issues all its loads (mask, then search strip) before the first use -- one L2 round
  // trip instead of a dependent one per row batch (cfg 4: 1.15 ms -> see DESIGN 6.2c per 8 pairs).
  const bool vec = (a.pitch & 3) == 0 && (x & 3) == 0 && ((x + a.mx) & 3) == 0 && (w & 3) == 0 &&
                   (reinterpret_cast<uintptr_t>(a.A) & 15) == 0 && (reinterpret_cast<uintptr_t>(Bf) & 15) == 0;
  if (vec) {
    constexpr int kTV = (TH * 16 + 511) / 512 + 1, kBV = ((TH + 72) * 16 + 511) / 512 + 1;
    const int w4 = w >> 2, lw4 = __ffs(w4) - 1, nT = TH * w4, nB = span * w4;  // w4 = 8 or 16
    float4 tv[kTV], bv[kBV];
#pragma unroll
    for (int k = 0; k < kTV; ++k) {
      const int e = tid + k * nth;
      if (e < nT) tv[k] = __ldg(reinterpret_cast<const float4*>(Aw + (int64_t)(e >> lw4) * a.pitch) + (e & (w4 - 1)));
    }
#pragma unroll
    for (int k = 0; k < kBV; ++k) {
      const int e = tid + k * nth;
      if (e < nB) bv[k] = __ldg(reinterpret_cast<const float4*>(Bw + (int64_t)(e >> lw4) * a.pitch) + (e & (w4 - 1)));
    }
#pragma unroll
    for (int k = 0; k < kTV; ++k)
      if (tid + k * nth < nT) s1 += ((double)tv[k].x + (double)tv[k].y) + ((double)tv[k].z + (double)tv[k].w);
#pragma unroll
    for (int k = 0; k < kBV; ++k) {
      const int e = tid + k * nth;
      if (e < nB) reinterpret_cast<float4*>(Bc)[e] = bv[k];
    }
    for (int e = nB * 4 + tid; e < (span + kBorderDY - 1) * w; e += nth) Bc[e] = 0.0f;
    // mean over the mask, then the centred mask stored straight from the registers (no second
    // pass over shared memory)
    s1 = warp_sum_d(s1);
    if (lane == 0) red[warp] = s1;
    __syncthreads();
    double tot = 0.0;
    for (int q = 0; q < nwarp; ++q) tot += red[q];
    const double mean = tot / ((double)TH * (double)w);
#pragma unroll
    for (int k = 0; k < kTV; ++k) {
      const int e = tid + k * nth;
      if (e < nT)
        reinterpret_cast<float4*>(T)[e] = make_float4((float)((double)tv[k].x - mean), (float)((double)tv[k].y - mean),
                                                      (float)((double)tv[k].z - mean), (float)((double)tv[k].w - mean));
    }
    __syncthreads();
  } else {
    for (int i = warp; i < TH; i += nwarp)
      for (int j = lane; j < w; j += 32) {
        const float v = __ldg(Aw + (int64_t)i * a.pitch + j);
        T[i * w + j] = v;
        s1 += (double)v;
      }
    for (int i = warp; i < span + kBorderDY - 1; i += nwarp)
      for (int j = lane; j < w; j += 32) Bc[i * w + j] = i < span ? __ldg(Bw + (int64_t)i * a.pitch + j) : 0.0f;
    s1 = warp_sum_d(s1);
    if (lane == 0) red[warp] = s1;
    __syncthreads();
    double tot = 0.0;
    for (int q = 0; q < nwarp; ++q) tot += red[q];
    const double mean = tot / ((double)TH * (double)w);
    for (int i = warp; i < TH; i += nwarp)
      for (int jj = lane; jj < w; jj += 32) T[i * w + jj] = (float)((double)T[i * w + jj] - mean);
    __syncthreads();
  }
  const int b = warp & 7, c = warp >> 3, j = 32 * c + lane, dy0 = kBorderDY * b;
  float tr[TH];  // the thread's template column, pinned in registers (volatile loads: not re-read per use)
#pragma unroll
  for (int i = 0; i < TH; ++i)
    asm volatile("ld.shared.f32 %0, [%1];" : "=f"(tr[i]) : "r"(smem_u32(T + i * w + j)));
  float acc[kBorderDY];
#pragma unroll
  for (int d = 0; d < kBorderDY; ++d) acc[d] = 0.0f;
  if (dy0 < OY) {
    const float* bcol = Bc + dy0 * w + j;
#pragma unroll
    for (int r = 0; r < TH + kBorderDY - 1; ++r) {
      const float xv = bcol[r * w];
#pragma unroll
      for (int d = 0; d < kBorderDY; ++d)
        if (r - d >= 0 && r - d < TH) acc[d] = fmaf(tr[r - d], xv, acc[d]);
    }
  }
#pragma unroll
  for (int d = 0; d < kBorderDY; ++d) {
    float v = acc[d];
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    if (lane == 0) part[(c * 8 + b) * kBorderDY + d] = v;
  }
  __syncthreads();
  for (int dy = tid; dy < OY; dy += nth) {
    float v = 0.0f;
    for (int cc = 0; cc < ncw; ++cc) v += part[(cc * 8 + dy / kBorderDY) * kBorderDY + dy % kBorderDY];
    const_cast<float*>(a.border)[((int64_t)z * a.Ky * a.Kx + lin) * OY + dy] = v;
  }
}

}  // namespace nccb
