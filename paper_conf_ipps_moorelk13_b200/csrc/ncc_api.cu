// ncc_api.cu -- C ABI (include/ncc.h) over the sm_100a kernels in ncc_kernels.cuh.
//
// Lifecycle follows GPU-PF: ncc_plan_create = specification +
// refresh (validate, choose the specialised variant, allocate scratch, set kernel
// attributes); ncc_match / piv_correlate = execution (launches only, no allocation);
// ncc_plan_destroy.  Variant selection (Ch. 4): problem
// parameters that control loop structure (template size, search radius) are baked into
// pre-instantiated kernels ("SK"); anything else runs the run-time-evaluated generic kernel
// ("RE").  Pointers and template values always stay run-time.
#include <cuda_runtime.h>

#include <dlfcn.h>
#include <sys/stat.h>
#include <sys/types.h>
#include <unistd.h>

#include <fstream>
#include <sstream>

#include <algorithm>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <new>
#include <string>
#include <mutex>
#include <vector>

#include "../../include/ncc.h"
#include "ncc_kernels.cuh"
#include "ncc_tc.cuh"
#include "ncc_sad.cuh"
#include "ncc_piv_tc.cuh"

using namespace nccb;

static_assert(sizeof(ncc_peak) == 16, "ncc_peak must be 16 B");
static_assert(sizeof(piv_vector) == 24, "piv_vector must be 24 B");
static_assert(sizeof(PeakOut) == sizeof(ncc_peak), "PeakOut layout");
static_assert(sizeof(VecOut) == sizeof(piv_vector), "VecOut layout");

namespace {

thread_local std::string g_last_cuda_error;

ncc_status cuda_fail(cudaError_t e, const char* where) {
  g_last_cuda_error = std::string(where) + ": " + cudaGetErrorString(e);
  return e == cudaErrorMemoryAllocation ? NCC_ERR_OUT_OF_MEMORY : NCC_ERR_CUDA;
}
#define NCC_CUDA(call)                                   \
  do {                                                   \
    cudaError_t _e = (call);                             \
    if (_e != cudaSuccess) return cuda_fail(_e, #call);  \
  } while (0)

// ------------------------------------------------------------------ variant tables
struct TmVariant {
  const char* name;
  int TH, TW;                 // 0 = run-time (RE)
  int RV, LX, WX, WY, CH, CW;
  const void* k[2][2];  // [tma][const template] kernels (AOT function or JIT cudaKernel_t)
  int smem[2][2];
  int nt, bu, bv, ir, ip;
  int rv_nt() const { return RV * nt; }
};

#define TM_K(RV, LX, WX, WY, CH, CW, TH, TW, TMA, CT) \
  reinterpret_cast<const void*>(&tm_ncc_kernel<RV, LX, WX, WY, CH, CW, TH, TW, TMA, CT>)
#define TM_VARIANT(NAME, TH, TW, RV, LX, WX, WY, CH, CW)                                                     \
  TmVariant {                                                                                             \
    NAME, TH, TW, RV, LX, WX, WY, CH, CW,                                                                 \
        {{TM_K(RV, LX, WX, WY, CH, CW, TH, TW, false, false), TM_K(RV, LX, WX, WY, CH, CW, TH, TW, false, true)}, \
         {TM_K(RV, LX, WX, WY, CH, CW, TH, TW, true, false), TM_K(RV, LX, WX, WY, CH, CW, TH, TW, true, true)}},  \
        {{TmTile<RV, LX, WX, WY, CH, CW>::smem_ldg(false), TmTile<RV, LX, WX, WY, CH, CW>::smem_ldg(true)},    \
         {TmTile<RV, LX, WX, WY, CH, CW>::smem_tma(false), TmTile<RV, LX, WX, WY, CH, CW>::smem_tma(true)}},   \
        TmTile<RV, LX, WX, WY, CH, CW>::NT, TmTile<RV, LX, WX, WY, CH, CW>::BU,                              \
        TmTile<RV, LX, WX, WY, CH, CW>::BV, TmTile<RV, LX, WX, WY, CH, CW>::IR,                              \
        TmTile<RV, LX, WX, WY, CH, CW>::IP                                                                   \
  }

const TmVariant kTmVariants[] = {
    // generic run-time-evaluated kernel (any h, w)
    TM_VARIANT("tm_re_rv12_lx4_4x1_c32x32", 0, 0, 12, 4, 1, 4, 32, 32),
    // specialised instances for the BASELINE configurations
    TM_VARIANT("tm_sk_16x16_rv4_lx16_4x1_c16x16", 16, 16, 4, 16, 1, 4, 16, 16),
    TM_VARIANT("tm_sk_128x128_rv12_lx4_4x1_c16x64", 128, 128, 12, 4, 1, 4, 16, 64),
    // alternative 128x128 tilings (selected with NCC_FORCE_VARIANT for sweeps)
    TM_VARIANT("tm_sk_128x128_rv12_lx4_4x1_c32x64", 128, 128, 12, 4, 1, 4, 32, 64),
    TM_VARIANT("tm_sk_128x128_rv12_lx4_8x1_c32x64", 128, 128, 12, 4, 1, 8, 32, 64),
    TM_VARIANT("tm_sk_128x128_rv12_lx4_4x2_c32x64", 128, 128, 12, 4, 2, 4, 32, 64),
    TM_VARIANT("tm_sk_128x128_rv12_lx4_8x1_c16x64", 128, 128, 12, 4, 1, 8, 16, 64),
    TM_VARIANT("tm_sk_512x512_rv12_lx4_4x1_c32x64", 512, 512, 12, 4, 1, 4, 32, 64),
};

// cuTensorMapEncodeTiled through the runtime's driver entry point (no -lcuda needed).
typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                  const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                  CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
EncodeTiledFn encode_fn() {
  static EncodeTiledFn fn = nullptr;
  static bool tried = false;
  if (!tried) {
    tried = true;
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<EncodeTiledFn>(p);
  }
  return fn;
}

// fp32 (or 8-byte element) tensor map of `rank` dims (innermost first), strides in bytes for dims 1..rank-1.
bool encode_f32(CUtensorMap* m, const void* base, int rank, const uint64_t* dims, const uint64_t* strides_bytes,
                const uint32_t* box, bool u64 = false) {
  EncodeTiledFn fn = encode_fn();
  if (!fn) return false;
  cuuint64_t gd[5], gs[4];
  cuuint32_t bx[5], es[5] = {1, 1, 1, 1, 1};
  for (int i = 0; i < rank; ++i) {
    gd[i] = dims[i];
    bx[i] = box[i];
  }
  for (int i = 0; i + 1 < rank; ++i) gs[i] = strides_bytes[i];
  return fn(m, u64 ? CU_TENSOR_MAP_DATA_TYPE_UINT64 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32, (cuuint32_t)rank,
            const_cast<void*>(base), gd, gs, bx, es,
            CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

constexpr int kTcColsMax = 8;  // ragged tensor-core column tiles up to this width run on tm_tc_cols

struct PivVariant {
  const char* name;
  int TH, TW, MY, MX;  // 0 = run-time (RE)
  int RV, CW, NT, WPB, ALIAS, IPT;
  const void* k_tma;  // AOT function or JIT cudaKernel_t
  const void* k_ldg;
  const void* k_ws = nullptr;  // persistent warp-specialised form (TMA only), if instantiated
  int ws_ncw = 0, ws_npw = 0;
  int ws_bp = 0;     // staged pitch (= TMA box width) of the WS kernel; 0: the plan's piv_bp
  int ws_bytes = 0;  // dynamic shared memory of the WS kernel; 0: 2 PivShape<12,64> stages + score tile
  int ws_wps = 1;    // windows per pipeline stage of the WS kernel
};
using Ws2Cfg4 = PivWs2Shape<64, 64, 32, 32, 16, 64, 1>;
using Ws2Cfg3 = PivWs2Shape<32, 32, 16, 16, 16, 32, 4>;
#define PIV_VARIANT_SK(NAME, TH, TW, MY, MX, RV, CW, NT, WPB, MINB, IPT)                                     \
  PivVariant {                                                                                              \
    NAME, TH, TW, MY, MX, RV, CW, NT, WPB, 1, IPT,                                                          \
        reinterpret_cast<const void*>(&piv_ncc_kernel<TH, TW, MY, MX, RV, CW, NT, WPB, MINB, true, true, IPT>),  \
        reinterpret_cast<const void*>(&piv_ncc_kernel<TH, TW, MY, MX, RV, CW, NT, WPB, MINB, false, true, IPT>)  \
  }
#define PIV_VARIANT_RE(NAME, RV, CW, NT, MINB)                                                              \
  PivVariant {                                                                                              \
    NAME, 0, 0, 0, 0, RV, CW, NT, 1, 0, 1,                                                                 \
        reinterpret_cast<const void*>(&piv_ncc_kernel<0, 0, 0, 0, RV, CW, NT, 1, MINB, true, false, 1>),       \
        reinterpret_cast<const void*>(&piv_ncc_kernel<0, 0, 0, 0, RV, CW, NT, 1, MINB, false, false, 1>)       \
  }

const PivVariant kPivVariants[] = {
    PIV_VARIANT_RE("piv_re_rv12_cw16_nt256", 12, 16, 256, 1),
    PivVariant{"piv_ws2_32x32_m16_rv16_c8p8_w4", 32, 32, 16, 16, 12, 32, 416, 4, 1, 1,
               reinterpret_cast<const void*>(&piv_ncc_kernel<32, 32, 16, 16, 12, 32, 416, 4, 2, true, true, 1>),
               reinterpret_cast<const void*>(&piv_ncc_kernel<32, 32, 16, 16, 12, 32, 416, 4, 2, false, true, 1>),
               reinterpret_cast<const void*>(&piv_ws2_kernel<32, 32, 16, 16, 16, 32, 8, 8, 4>), 8, 8, Ws2Cfg3::BP,
               Ws2Cfg3::smem_bytes, 4},
    PIV_VARIANT_SK("piv_sk_32x32_m16_rv12_nt416_w4", 32, 32, 16, 16, 12, 32, 416, 4, 2, 1),
    PivVariant{"piv_ws2_64x64_m32_rv16_c8p8", 64, 64, 32, 32, 12, 64, 416, 1, 1, 1,
               reinterpret_cast<const void*>(&piv_ncc_kernel<64, 64, 32, 32, 12, 64, 416, 1, 2, true, true, 1>),
               reinterpret_cast<const void*>(&piv_ncc_kernel<64, 64, 32, 32, 12, 64, 416, 1, 2, false, true, 1>),
               reinterpret_cast<const void*>(&piv_ws2_kernel<64, 64, 32, 32, 16, 64, 8, 8, 1>), 8, 8, Ws2Cfg4::BP,
               Ws2Cfg4::smem_bytes, 1},
    PivVariant{"piv_ws_64x64_m32_rv12_c13p4", 64, 64, 32, 32, 12, 64, 416, 1, 1, 1,
               reinterpret_cast<const void*>(&piv_ncc_kernel<64, 64, 32, 32, 12, 64, 416, 1, 2, true, true, 1>),
               reinterpret_cast<const void*>(&piv_ncc_kernel<64, 64, 32, 32, 12, 64, 416, 1, 2, false, true, 1>),
               reinterpret_cast<const void*>(&piv_ws_kernel<64, 64, 32, 32, 12, 64, 13, 4>), 13, 4},
    PIV_VARIANT_SK("piv_sk_64x64_m32_rv12_nt416_w1", 64, 64, 32, 32, 12, 64, 416, 1, 2, 1),
    // alternatives with warp counts that are multiples of 4 (even SMSP load; NCC_FORCE_VARIANT)
    PIV_VARIANT_SK("piv_sk_64x64_m32_rv12_nt512_w1", 64, 64, 32, 32, 12, 64, 512, 1, 2, 1),
    PIV_VARIANT_SK("piv_sk_32x32_m16_rv12_nt512_w5", 32, 32, 16, 16, 12, 32, 512, 5, 1, 1),
    PIV_VARIANT_SK("piv_sk_32x32_m16_rv12_nt512_w4", 32, 32, 16, 16, 12, 32, 512, 4, 2, 1),
};

constexpr int kBoxRowsNT = 256, kBoxRowsSEG = 2048;  // max segment; actual = min(V, SEG)
constexpr int kBoxColsNW = 8, kBoxColsL = 16;  // 32 columns x 8 warps x 16 rows per CTA
constexpr int kBox2dNT = 256, kBoxTV = 128;      // fused window sums: 128-column strips

int ceil_div(int64_t a, int64_t b) { return (int)((a + b - 1) / b); }

// The 64 KB constant-bank template slot (c_tpl) is one per device.  Every writer orders itself
// after the previous user on any stream with a per-device event, so concurrent TM plans on
// different streams of one device stay correct (they serialise on the slot, nothing else).
struct ConstSlot {
  std::mutex mu;
  cudaEvent_t done = nullptr;
};
ConstSlot g_const_slot[64];

// Run-time mirror of TmTile<> (same formulas) for run-time specialised variants.
TmVariant tm_geom(int RV, int LX, int WX, int WY, int CH, int CW) {
  TmVariant v{};
  v.RV = RV; v.LX = LX; v.WX = WX; v.WY = WY; v.CH = CH; v.CW = CW;
  v.nt = WX * WY * 32;
  v.bu = WY * (32 / LX);
  v.bv = WX * LX * RV;
  v.ir = v.bu + CH - 1;
  v.ip = pick_pitch(v.bv + CW, RV, LX);
  const int tb = CH * CW * 4, ib = v.ir * v.ip * 4;
  const int tal = ((tb + 127) / 128) * 128, ial = ((ib + 127) / 128) * 128;
  v.smem[0][0] = tb + ib;
  v.smem[0][1] = ib;
  v.smem[1][0] = 2 * (tal + ial);
  v.smem[1][1] = 2 * ial;
  return v;
}

// Smallest-padding chunk width / height from the candidates (ties -> the larger chunk).
int pick_chunk(int n, const int* cands, int nc) {
  int best = cands[0], bp = 1 << 30;
  for (int i = 0; i < nc; ++i) {
    const int pad = ((n + cands[i] - 1) / cands[i]) * cands[i] - n;
    if (pad < bp) { bp = pad; best = cands[i]; }
  }
  return best;
}

struct TmJitChoice {
  int RV, LX, WX, WY, CH, CW;
  bool ct;
};
// NCC_TM_JIT="RV,LX,WX,WY,CH,CW" forces a run-time specialised tile (the Tab 6.21 sensitivity
// sweep, tools/sensitivity.py); the AOT instance for (h, w) is then skipped too.
bool tm_jit_forced(TmJitChoice* c) {
  const char* e = getenv("NCC_TM_JIT");
  if (!e) return false;
  int v[6];
  if (sscanf(e, "%d,%d,%d,%d,%d,%d", &v[0], &v[1], &v[2], &v[3], &v[4], &v[5]) != 6) return false;
  if (c) *c = TmJitChoice{v[0], v[1], v[2], v[3], v[4], v[5], false};
  return true;
}
TmJitChoice tm_jit_choice(int h, int w) {
  static const int cw[] = {64, 32, 16}, ch[] = {32, 16};
  TmJitChoice c{12, 4, 1, 4, pick_chunk(h, ch, 2), pick_chunk(w, cw, 3), false};
  tm_jit_forced(&c);
  const int WP = ((w + c.CW - 1) / c.CW) * c.CW;
  c.ct = (kConstTplFloats / WP) / c.CH * c.CH >= c.CH;
  return c;
}

struct PivJitChoice {
  int RV, CW, NT, WPB, MINB, BP, items;
  int64_t win_fl;
  bool ok;
};
// Run-time mirror of PivShape<RV, CW> (same formulas): items and per-window floats.
struct PivShapeRT {
  int items;
  int64_t win_fl;
};
PivShapeRT piv_shape_rt(int RV, int CW, int h, int w, int my, int mx, int BP, bool alias) {
  const int OY = 2 * my + 1, OX = 2 * mx + 1, OXP = ((OX + RV - 1) / RV) * RV;
  const int TPP = ((w + CW - 1) / CW) * (CW + 2), BR = h + 2 * my;
  const int64_t tp_fl = (((int64_t)h * TPP * 2 + 31) / 32) * 32, b_fl = (((int64_t)BR * BP + 31) / 32) * 32;
  const int64_t s_fl = (((int64_t)OY * OXP + 31) / 32) * 32;
  return PivShapeRT{OY * ((OX + RV - 1) / RV), (alias ? std::max(tp_fl, s_fl) : tp_fl + s_fl) + b_fl};
}
PivJitChoice piv_jit_choice(int h, int w, int my, int mx) {
  static const int cw[] = {64, 32, 16};
  PivJitChoice c{};
  c.RV = 12;
  int force_wpb = 0;  // NCC_PIV_JIT="RV,WPB": the Tab 6.22 sensitivity sweep (data registers x threads)
  if (const char* e = getenv("NCC_PIV_JIT")) {
    int rv = 0, wpb = 0;
    if (sscanf(e, "%d,%d", &rv, &wpb) == 2 && rv >= 4 && rv % 4 == 0 && wpb >= 1) {
      c.RV = rv;
      force_wpb = wpb;
    }
  }
  c.CW = pick_chunk(w, cw, 3);
  const int OX = 2 * mx + 1, NG = (OX + c.RV - 1) / c.RV;
  c.BP = piv_pick_pitch(NG * c.RV + ((w + c.CW - 1) / c.CW) * c.CW, c.RV, NG);
  const PivShapeRT ps = piv_shape_rt(c.RV, c.CW, h, w, my, mx, c.BP, true);
  const int items = ps.items;
  c.win_fl = ps.win_fl;
  c.items = items;
  c.ok = false;
  if (items > 1024) return c;  // one item per thread (score tile aliased on the template pairs)
  const int64_t kTwoPerSm = 113 * 1024, kOnePerSm = 227 * 1024;
  if (force_wpb) {  // sweeps: exactly the requested windows per CTA
    const int nt = ((force_wpb * items + 31) / 32) * 32;
    const int64_t smem = (int64_t)force_wpb * c.win_fl * 4;
    if (nt > 1024 || smem > kOnePerSm) return c;
    c.WPB = force_wpb;
    c.NT = nt;
    c.MINB = smem <= kTwoPerSm ? 2 : 1;
    c.ok = true;
    return c;
  }
  double best = -1.0;
  // One window per CTA unless its items fill under 60 % of the warps: the Tab 6.22 surface
  // (EXPERIMENTS.md, cfg3 shape) puts WPB = 1 first at every RV (k = 3 / 4: 86-90 %) -- more
  // windows per CTA blow up the per-window register arrays (48^2 / 64^2 masks: 128-138 registers,
  // slower than the generic kernel).
  const double util1 = (double)items / (((items + 31) / 32) * 32);
  const int kmax = util1 >= 0.6 ? 1 : 4;
  for (int k = 1; k <= kmax; ++k) {
    if (force_wpb && k != force_wpb) continue;
    const int nt = ((k * items + 31) / 32) * 32;
    const int64_t smem = (int64_t)k * c.win_fl * 4;
    if (nt > 1024 || smem > kOnePerSm) break;
    double util = (double)(k * items) / nt;
    if (smem <= kTwoPerSm) util += 0.05;  // prefer two resident CTAs per SM (phase overlap)
    if (util > best + 1e-9) {
      best = util;
      c.WPB = k;
      c.NT = nt;
      c.MINB = smem <= kTwoPerSm ? 2 : 1;
      c.ok = true;
    }
  }
  return c;
}

#include "ncc_jit.inc"

}  // namespace

// ------------------------------------------------------------------ plan object
struct ncc_plan_s {
  ncc_problem p;
  int device;
  ncc_plan_info info;
  // TM
  int U, V, u_begin, u_end, Ub, Hs, HP, WP;
  int tiles_u, tiles_v, split;
  int n_tmpl;     // templates per frame (ROI mode) or 1
  bool roi_mode;
  bool tma_ok;
  int use_ct, slab_rows, n_slabs;  // constant-template slabs (rows per slab, slab count)
  float* carry;
  CUtensorMap map_tpl;
  float* part;
  unsigned int* cnt;
  const TmVariant* tmv;
  TmVariant tmv_store;  // run-time specialised variant
  PivVariant pivv_store;
  cudaLibrary_t jit_lib;
  void* jit_ctpl;  // the JIT library's own constant-bank template slot (nullptr: AOT, global slot)
  double jit_ms;   // NVRTC compile time (0 when loaded from the cache)
  int jit_ct;      // JIT TM: template mode compiled (1 = constant bank)
  char jit_name[96];
  float* tplC;
  TemplateStats* tst;
  unsigned long long* keys;
  // PIV
  int Ky, Kx, OY, OX, sub_batch, host_chunk, piv_bp, piv_smem, map_w, map_h;
  int ws_smem, ws_grid;  // persistent warp-specialised PIV kernel (0: not used)
  int ws_bp;             // its staged pitch = TMA box width
  const PivVariant* pivv;
  // tensor-core PIV numerator (piv_tc_kernel; 0: CUDA cores): rows per MMA, smem, grid, strip segments
  int ptc, ptc_R, ptc_smem, ptc_border_smem, ptc_nseg, ptc_segw, ptc_border_rb;
  float* ptc_border;     // [sub_batch][Ky Kx][OY] numerators of the last column (piv_tc_border_kernel)
  unsigned long long* ptc_prof;  // NCC_PIV_TC_PROF=<file>: per-CTA wait accounting, dumped at destroy
  // shared scratch (window sums)
  double *RS1, *RS2, *S1, *S2;
  int64_t rs_frame_stride, s_frame_stride;
  int box_r, box_iwp, box_smem, nsm;  // fused window-sum kernel (box_smem 0: two-pass fallback)
  float* tc_img2 = nullptr;  // band rows as the tensor-core numerator's image operand (tm_tc_split)
  // tensor-core numerator (tm_tc_kernel): 0 = CUDA-core path
  int tc, tc_wc, tc_nbi, tc_nbj, tc_vtiles, tc_useg, tc_nseg;
  int tc_vcols;  // last output columns computed by tm_tc_cols (0: none)
  int tc_sched;  // 0: window sums || template prep, image split after them; 3 (default): image split,
                 // then window sums || template prep + ragged columns
  float *tcB, *tc_acc;     // reversed template-block operands; running numerator (one plane, chain mode)
  int tc_planes;           // planes mode (few template blocks): per-block partial planes + tm_tc_finish
  int tc_clen, tc_nplanes; // blocks per chain (1: planes, nblk: one chain), planes tm_tc_finish sums
  int tc_box_late;         // planes mode: window sums after the numerator, as its programmatic dependent
  float* tc_part;          // [nblk][batch][Ub][V] partial numerators (planes mode)
  unsigned int* tc_done;   // finished tm_tc_tail CTAs (self-resetting)
  unsigned int* tc_flags;  // chain flags [batch][vtiles * nseg][ngrp_max][4] (self-resetting)
  unsigned long long* tc_ticket;  // CTA start tickets (monotonic)
  int tc_ngrp;
  int tc_exp;  // NCC_TC_EXP timing experiments (0 in normal use; results are wrong with bits set)
  int tc_center;  // image operand centred on the template mean (NCC_TC_CENTER=0/1)
  unsigned long long* tc_prof;  // NCC_TC_EXP bit 32: per-CTA wait accounting (tools/tc_prof.py)
  float *tc_rsv, *tc_mean;  // NCC tensor-core plans: fp32 rsqrt(n var) and window mean per offset (window-sum kernels)
  int sad, sad_smem;  // NCC_SCORE_SAD: the direct |t - b| kernels (ncc_sad.cuh), their dynamic smem
  // tiny problems: the whole TM path in one launch (tm_tiny_kernel)
  const void* tiny_fn;
  int tiny_ctas, tiny_rows, tiny_smem;
  unsigned int* tiny_done;
  // side stream for work independent of the main chain (template prep || window sums)
  cudaStream_t side, side2;  // side2: the window sums beside the numerator (TM schedule 5)
  cudaEvent_t ev_box;
  cudaEvent_t ev_fork, ev_join, ev_cols, ev_img;
  // timing (NCC_F_TIMING)
  std::vector<cudaEvent_t> ev;
  int n_ev_used;
  int timing_kind;  // 0 none, 1 TM, 2 PIV
  int piv_nsub;
  // host staging (lazy)
  float *st_a, *st_b, *st_t, *st_s;
  void* st_out;
  size_t st_a_bytes, st_b_bytes, st_t_bytes, st_s_bytes, st_out_bytes;
  // PIV host streaming (lazy): copy stream, per-slot "copied" / "slot free" events
  cudaStream_t copy;
  cudaEvent_t ev_copied[2], ev_free[2], ev_start;
  // CUDA-graph replay of execute calls (lazy): capture stream, a few instantiated graphs keyed
  // by the call's pointer arguments (the host path alternates two staging slots)
  cudaStream_t cap;
  int capturing;
  // host path (ncc_match_host): inputs copied inside the launch sequence -- the template on the
  // side stream ahead of its prep, the frames on the main stream -- so the prep overlaps the
  // frames' copy (transient, set around one call)
  const float* h_img_in;
  const float* h_tmpl_in;
  int64_t h_tmpl_pitch;
  struct GraphEntry {
    uintptr_t key[8];
    cudaGraphExec_t exec;
    int timing_kind, piv_nsub;  // host-side facts of the captured sequence, restored on replay
  } graphs[4];
  int n_graphs, next_graph;
};

namespace {

struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    if (cudaGetDevice(&prev) == cudaSuccess && prev != dev) cudaSetDevice(dev);
    else prev = -1;
  }
  ~DeviceGuard() {
    if (prev >= 0) cudaSetDevice(prev);
  }
};

void free_plan(ncc_plan pl) {
  if (pl->ptc_prof) {
    if (const char* path = getenv("NCC_PIV_TC_PROF")) {
      std::vector<unsigned long long> h((size_t)pl->nsm * 32 + 3 * 2048);
      if (cudaMemcpy(h.data(), pl->ptc_prof, h.size() * 8, cudaMemcpyDeviceToHost) == cudaSuccess)
        if (FILE* fp = fopen(path, "wb")) {
          fwrite(h.data(), 8, h.size(), fp);
          fclose(fp);
        }
    }
  }
  cudaFree(pl->ptc_prof);
  if (pl->tc_prof) {  // NCC_TC_EXP bit 32: the per-CTA accounting of the last call to NCC_TC_PROF_DUMP
    if (const char* path = getenv("NCC_TC_PROF_DUMP")) {
      const size_t n = (size_t)pl->tc_nbi * pl->tc_nbj * pl->tc_vtiles * pl->tc_nseg * pl->p.batch * 8 + 512;
      std::vector<unsigned long long> h(n);
      if (cudaMemcpy(h.data(), pl->tc_prof, n * 8, cudaMemcpyDeviceToHost) == cudaSuccess)
        if (FILE* fp = fopen(path, "wb")) {
          fwrite(h.data(), 8, n, fp);
          fclose(fp);
        }
    }
  }
  cudaFree(pl->tplC);
  cudaFree(pl->part);
  cudaFree(pl->cnt);
  cudaFree(pl->carry);
  cudaFree(pl->tst);
  cudaFree(pl->keys);
  cudaFree(pl->RS1);
  cudaFree(pl->tcB);
  cudaFree(pl->tc_acc);
  cudaFree(pl->tc_part);
  cudaFree(pl->tc_done);
  cudaFree(pl->tc_flags);
  cudaFree(pl->tc_ticket);
  cudaFree(pl->tc_prof);
  cudaFree(pl->tc_rsv);
  cudaFree(pl->tc_mean);
  cudaFree(pl->ptc_border);
  cudaFree(pl->tiny_done);
  cudaFree(pl->tc_img2);
  cudaFree(pl->RS2);
  cudaFree(pl->S1);
  cudaFree(pl->S2);
  cudaFree(pl->st_a);
  cudaFree(pl->st_b);
  cudaFree(pl->st_t);
  cudaFree(pl->st_s);
  cudaFree(pl->st_out);
  for (cudaEvent_t e : pl->ev) cudaEventDestroy(e);
  if (pl->ev_fork) cudaEventDestroy(pl->ev_fork);
  if (pl->ev_join) cudaEventDestroy(pl->ev_join);
  if (pl->ev_cols) cudaEventDestroy(pl->ev_cols);
  if (pl->ev_img) cudaEventDestroy(pl->ev_img);
  if (pl->side) cudaStreamDestroy(pl->side);
  if (pl->side2) cudaStreamDestroy(pl->side2);
  if (pl->ev_box) cudaEventDestroy(pl->ev_box);
  for (int k = 0; k < 2; ++k) {
    if (pl->ev_copied[k]) cudaEventDestroy(pl->ev_copied[k]);
    if (pl->ev_free[k]) cudaEventDestroy(pl->ev_free[k]);
  }
  if (pl->ev_start) cudaEventDestroy(pl->ev_start);
  if (pl->copy) cudaStreamDestroy(pl->copy);
  for (int k = 0; k < pl->n_graphs; ++k)
    if (pl->graphs[k].exec) cudaGraphExecDestroy(pl->graphs[k].exec);
  if (pl->cap) cudaStreamDestroy(pl->cap);
  if (pl->jit_lib) cudaLibraryUnload(pl->jit_lib);
  delete pl;
}

ncc_status validate(const ncc_problem& p) {
  if (p.score != NCC_SCORE_NCC && p.score != NCC_SCORE_SSD && p.score != NCC_SCORE_SAD) return NCC_ERR_INVALID_ARGUMENT;
  if (p.mode != NCC_MODE_MATCH && p.mode != NCC_MODE_PIV) return NCC_ERR_INVALID_ARGUMENT;
  if (p.image_h <= 0 || p.image_w <= 0 || p.tmpl_h <= 0 || p.tmpl_w <= 0) return NCC_ERR_INVALID_ARGUMENT;
  if (p.image_pitch < p.image_w) return NCC_ERR_INVALID_ARGUMENT;
  if (p.tmpl_h > p.image_h || p.tmpl_w > p.image_w) return NCC_ERR_INVALID_ARGUMENT;
  if (p.batch < 1 || p.shard_count < 1 || p.shard_rank < 0 || p.shard_rank >= p.shard_count)
    return NCC_ERR_INVALID_ARGUMENT;
  if (p.n_templates < 0 || p.roi_h < 0 || p.roi_w < 0) return NCC_ERR_INVALID_ARGUMENT;
  if (p.mode == NCC_MODE_MATCH) {
    if (p.search_y != 0 || p.search_x != 0) return NCC_ERR_INVALID_ARGUMENT;
    if (p.roi_h > 0 || p.roi_w > 0 || p.n_templates > 1) {  // ROI mode
      if (p.roi_h < 1 || p.roi_w < 1 || p.n_templates < 1 || p.shard_count != 1) return NCC_ERR_INVALID_ARGUMENT;
      if (p.roi_h > p.image_h - p.tmpl_h + 1 || p.roi_w > p.image_w - p.tmpl_w + 1) return NCC_ERR_INVALID_ARGUMENT;
    }
    const int64_t U = p.image_h - p.tmpl_h + 1, V = p.image_w - p.tmpl_w + 1;
    if (U * V >= (int64_t)0xFFFFFFF0ll) return NCC_ERR_INVALID_ARGUMENT;  // 32-bit key index
    if (p.shard_count > U) return NCC_ERR_INVALID_ARGUMENT;               // every band has rows
  } else {
    if (p.search_y < 0 || p.search_x < 0 || p.step_y <= 0 || p.step_x <= 0) return NCC_ERR_INVALID_ARGUMENT;
    if (p.image_h - p.tmpl_h - 2 * p.search_y < 0 || p.image_w - p.tmpl_w - 2 * p.search_x < 0)
      return NCC_ERR_INVALID_ARGUMENT;
    if (p.shard_count != 1 || p.shard_rank != 0) return NCC_ERR_INVALID_ARGUMENT;
    if (p.subpix < 0 || p.subpix > 2) return NCC_ERR_INVALID_ARGUMENT;
    if (p.n_templates > 1 || p.roi_h > 0 || p.roi_w > 0) return NCC_ERR_INVALID_ARGUMENT;
  }
  return NCC_OK;
}

template <class T>
ncc_status dalloc(T** ptr, size_t count) {
  *ptr = nullptr;
  if (count == 0) return NCC_OK;
  cudaError_t e = cudaMalloc((void**)ptr, count * sizeof(T));
  if (e != cudaSuccess) {
    *ptr = nullptr;
    return cuda_fail(e, "cudaMalloc");
  }
  return NCC_OK;
}

void fill_kernel_info(ncc_plan pl, const void* fn, int nt, int smem, int gx, int gy, int gz) {
  cudaFuncAttributes fa;
  if (cudaFuncGetAttributes(&fa, fn) == cudaSuccess) pl->info.regs_per_thread = fa.numRegs;
  pl->info.threads_per_block = nt;
  pl->info.smem_per_block = smem;
  pl->info.grid_x = gx;
  pl->info.grid_y = gy;
  pl->info.grid_z = gz;
}

// Fused window-sum kernel geometry: R rows of a (kBoxTV + w - 1)-column strip staged per
// sub-block; NCC_BOX_TWO_PASS=1 (or a strip too wide for shared memory) keeps the two-pass form.
ncc_status setup_box(ncc_plan pl, int w) {
  int maxsm = 0;
  NCC_CUDA(cudaDeviceGetAttribute(&maxsm, cudaDevAttrMaxSharedMemoryPerBlockOptin, pl->device));
  NCC_CUDA(cudaDeviceGetAttribute(&pl->nsm, cudaDevAttrMultiProcessorCount, pl->device));
  {  // padded row: 32 chunks of L (power of two) columns + one pad double per chunk
    int L = 1;
    while (32 * L < kBoxTV + w - 1) L *= 2;
    pl->box_iwp = 32 * L + 32;
  }
  const int64_t r = ((int64_t)maxsm / 8 - 2 * pl->box_iwp) / (2 * pl->box_iwp);
  pl->box_r = r > 16 ? 16 : (int)r;
  pl->box_smem = 0;
  // the fused form re-sums h - 1 halo rows and w - 1 halo columns per CTA: for large windows
  // (cfg 5: 512^2, ~45 loads per output) the two-pass form (row prefix sums, then a column
  // scan; ~3 loads per output) is 3.3x faster (834 -> 251 us, measured); below 256 the fused
  // form wins or ties (cfg 2: 18 vs 17.5 us, PIV 32^2: 16 us)
  const bool large = (pl->p.tmpl_h >= 256 || w >= 256) && !getenv("NCC_BOX_FUSED");  // NCC_BOX_FUSED=1: tests
  if (pl->box_r >= 1 && !large && !getenv("NCC_BOX_TWO_PASS")) {
    pl->box_smem = (2 * pl->box_r + 2) * pl->box_iwp * (int)sizeof(double);
    NCC_CUDA(cudaFuncSetAttribute((const void*)box2d_kernel<kBox2dNT>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                  pl->box_smem));
  }
  return NCC_OK;
}

// Tensor-core numerator (ncc_tc.cuh) for band-mode TM: template blocks of tc::kHB rows x WC
// columns, 128-column output tiles, output-row segments.  WC and the segment count minimise
// waves x (image rows per CTA) x (column chunks per row), the kernel's MMA time model.
ncc_status setup_tc(ncc_plan pl) {
  const ncc_problem& p = pl->p;
  pl->tc = 0;
  // NCC_TC=0 / NCC_F_CUDA_CORES / generic plans: CUDA-core path; NCC_TC=1: tensor cores whenever
  // eligible; default: the cost model below (tensor cores when clearly faster).
  const char* env = getenv("NCC_TC");
  const int mode = env ? atoi(env) : -1;
  if (mode == 0 || (p.flags & (NCC_F_CUDA_CORES | NCC_F_GENERIC_KERNEL)) || (!pl->roi_mode && pl->n_tmpl != 1))
    return NCC_OK;
  const int h = p.tmpl_h, w = p.tmpl_w;
  // ROI / multi-template mode: every (frame, template) pair is a sub-problem of roi_h x
  // roi_w offsets whose origin the kernel reads at run time; planes mode only, no ragged-column kernel
  const bool roi = pl->roi_mode;
  const int rows = roi ? p.roi_h : pl->Ub, cols = roi ? p.roi_w : pl->V;
  const int nsub = p.batch * (roi ? pl->n_tmpl : 1);
  // a ragged last column tile of at most kTcColsMax columns goes to tm_tc_cols instead of a
  // whole column of tensor-core CTAs
  pl->tc_vtiles = ceil_div(roi ? cols + 3 : cols, 128);  // ROI tiles start at the column <= the origin that is a multiple of 4
  pl->tc_vcols = 0;
  // launch order (measured on B200, cfg2 step: 0 -> 0.2135 ms, 3 -> 0.2074 ms; 1/2 delay the
  // tensor-core kernel's start or starve the ragged-column kernel); NCC_TM_SCHED overrides
  pl->tc_sched = getenv("NCC_TM_SCHED") ? atoi(getenv("NCC_TM_SCHED")) : 3;
  if (pl->tc_sched != 0 && pl->tc_sched != 4 && pl->tc_sched != 5 && pl->tc_sched != 6) pl->tc_sched = 3;  // (1/2: retired)
  if (!roi && pl->V > 128 && pl->V % 128 != 0 && pl->V % 128 <= kTcColsMax && w <= 512 && !getenv("NCC_TC_NO_COLS")) {
    pl->tc_vtiles = pl->V / 128;
    pl->tc_vcols = pl->V % 128;
  }
  pl->tc_nbi = ceil_div(h, tc::kHB);
  double best = 1e300;
  // WC = 32 unless forced (NCC_TC_WC, sweeps): the tensor cores' fp32 accumulation is biased
  // (truncating) -- at a planted peak, where every product is positive, the relative error of a
  // block's sum grows with its accumulation count (128 rows x WC/8 K-steps x 3): measured max
  // |dNCC| 2.25e-5 at WC = 32 and 4.6e-5 at WC = 64 (tools/tc_error.py, cfg2 / cfg5), so the
  // wider blocks would spend most of the 1e-4 budget.
  const int force_wc = getenv("NCC_TC_WC") ? atoi(getenv("NCC_TC_WC")) : tc::kWB;
  for (int wc = tc::kWB; wc <= 128; wc *= 2) {
    if (force_wc && wc != force_wc) {
      if (wc >= w) break;
      continue;
    }
    const int nbj = ceil_div(w, wc);
    const int64_t per_seg = (int64_t)pl->tc_vtiles * pl->tc_nbi * nbj * nsub;
    const int force_seg = getenv("NCC_TC_NSEG") ? atoi(getenv("NCC_TC_NSEG")) : 0;  // sweeps
    for (int nseg = 1; nseg <= 64 && nseg <= rows; ++nseg) {
      if (force_seg > 0 && nseg != force_seg) continue;
      const int useg = ceil_div(rows, nseg);
      const int64_t ctas = per_seg * ceil_div(rows, useg);
      const int64_t waves = (ctas + pl->nsm - 1) / pl->nsm;
      // cycles of a CTA: per stage ~320 cycles of fixed cost + 12 MMAs of 68 x N/136 cycles,
      // N = the group's trimmed window (tm_tc_kernel: ramp-in / ramp-out rows cover fewer columns)
      double cta = 0.0;
      const int ngrp = ceil_div(useg + tc::kHB - 1, tc::kG);
      for (int g = 0; g < ngrp; ++g) {
        const int lo = std::max(0, tc::kHB - 1 - tc::kG * g);
        const int chi = std::min(tc::kNWin, useg + tc::kHB - 1 - tc::kG * g);
        const int c0 = (lo / 8) * 8;
        const int n = std::max(16, ((chi - c0 + 7) / 8) * 8);
        cta += tc::kG * (320.0 + 12.0 * 68.0 * n / tc::kNWin);
      }
      const double cost = (double)waves * cta * (wc / tc::kWB);
      if (cost < best * 0.98) {  // more segments only when clearly cheaper (per-CTA setup is not modelled)
        best = cost;
        pl->tc_wc = wc;
        pl->tc_nbj = nbj;
        pl->tc_useg = useg;
        pl->tc_nseg = ceil_div(rows, useg);
      }
    }
    if (wc >= w) break;
  }
  // measured B200 rates: ~1050-1170 cycles per full tensor-core stage (12 MMAs of 128 x 136 x 8,
  // 3xTF32; modelled above), ~95 useful FP32 MACs per cycle per SM on the CUDA-core path
  const double tc_cycles = best;
  const double cc_cycles = (double)h * w * (double)rows * cols * nsub / (95.0 * pl->nsm);
  if (mode < 0 && !(tc_cycles < 0.8 * cc_cycles)) return NCC_OK;
  const int nblk = pl->tc_nbi * pl->tc_nbj;
  ncc_status st;
  if ((st = dalloc(&pl->tcB, (size_t)pl->n_tmpl * nblk * (tc::b_bytes(pl->tc_wc) / 4)))) return st;
  // Few template blocks (cfg2: 4): each block writes its own partial plane (no waiting between
  // CTAs) and tm_tc_finish sums them in block order.  Many (cfg5: 64): "chained planes" -- chains of
  // ceil(nblk / 16) consecutive blocks accumulate in-kernel (block b adds its sums to the running
  // numerator block b - 1 of its chain published), each chain's last block writes one plane, and
  // tm_tc_finish sums the <= 16 planes in order: per output ((p_0 + p_1) + ...) in block order, as
  // in both pure forms.  Measured at cfg5 (ms per step): one 64-block chain 19.4-20.3 (every CTA
  // waits for its predecessors' start-up), 64 planes 18.3 (3.4 GB of writes), chains of 16 / 8 / 4
  // blocks 18.8 / 18.8 / 18.3 (0.2 / 0.4 / 0.8 GB).  NCC_TC_PLANES=0 (one chain) / 1 (pure planes)
  // and NCC_TC_CLEN override.
  pl->tc_planes = 1;
  pl->tc_clen = nblk <= 8 ? 1 : ceil_div(nblk, 16);
  if (const char* e = getenv("NCC_TC_PLANES")) {
    pl->tc_planes = atoi(e) != 0;
    pl->tc_clen = pl->tc_planes ? 1 : nblk;
  }
  if (const char* e = getenv("NCC_TC_CLEN")) pl->tc_clen = std::max(1, std::min(nblk, atoi(e)));
  if (roi) {  // ROI mode: planes (small per-ROI planes, any block count)
    pl->tc_planes = 1;
    pl->tc_clen = 1;
  }
  pl->tc_nplanes = ceil_div(nblk, pl->tc_clen);
  pl->tc_box_late = getenv("NCC_TC_BOX_LATE") ? atoi(getenv("NCC_TC_BOX_LATE")) : 0;  // measured: slower
  if (pl->tc_planes && (st = dalloc(&pl->tc_part, (size_t)pl->tc_nplanes * nsub * rows * cols))) return st;
  if ((pl->tc_clen > 1 || !pl->tc_planes) &&  // running numerators: one plane per chain
      (st = dalloc(&pl->tc_acc, (size_t)pl->tc_nplanes * p.batch * pl->Ub * pl->V)))
    return st;
  pl->tc_ngrp = ceil_div(pl->tc_useg + tc::kHB - 1, tc::kG);
  pl->tc_exp = getenv("NCC_TC_EXP") ? atoi(getenv("NCC_TC_EXP")) : 0;
  pl->tc_center = getenv("NCC_TC_CENTER") ? atoi(getenv("NCC_TC_CENTER")) : 0;
  if (pl->tc_exp & 32) {
    const size_t n = (size_t)nblk * pl->tc_vtiles * pl->tc_nseg * nsub * 8 + 512;  // + group traces
    if ((st = dalloc(&pl->tc_prof, n))) return st;
    NCC_CUDA(cudaMemset(pl->tc_prof, 0, n * 8));
  }
  const size_t nflags = (size_t)p.batch * pl->tc_vtiles * pl->tc_nseg * pl->tc_nplanes * pl->tc_ngrp * 4;
  if ((st = dalloc(&pl->tc_flags, nflags))) return st;
  NCC_CUDA(cudaMemset(pl->tc_flags, 0, nflags * sizeof(unsigned int)));
  if ((st = dalloc(&pl->tc_ticket, (size_t)1))) return st;
  NCC_CUDA(cudaMemset(pl->tc_ticket, 0, sizeof(unsigned long long)));
  // image operand (tm_tc_split): per band row two planes of ((W + 1) & ~1) 8-byte elements
  if ((st = dalloc(&pl->tc_img2, (size_t)p.batch * pl->Hs * 4 * ((p.image_w + 1) & ~1)))) return st;
  if (p.score == NCC_SCORE_NCC) {  // per-offset fp32 normalisation factors (window-sum kernels)
    if ((st = dalloc(&pl->tc_rsv, (size_t)p.batch * pl->s_frame_stride))) return st;
    if ((st = dalloc(&pl->tc_mean, (size_t)p.batch * pl->s_frame_stride))) return st;
  }
  if ((st = dalloc(&pl->tc_done, (size_t)1))) return st;
  NCC_CUDA(cudaMemset(pl->tc_done, 0, sizeof(unsigned int)));
  const int smem = tc::smem_bytes(pl->tc_wc);
  NCC_CUDA(cudaFuncSetAttribute((const void*)tm_tc_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  NCC_CUDA(cudaFuncSetAttribute((const void*)tm_tc_prep, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                kPrepSmemFloats * 4));
  pl->tc = 1;
  ncc_plan_info& in = pl->info;
  char mode_s[24];
  if (!pl->tc_planes) snprintf(mode_s, sizeof(mode_s), "chain");
  else if (pl->tc_clen == 1) snprintf(mode_s, sizeof(mode_s), "planes");
  else snprintf(mode_s, sizeof(mode_s), "chain%d_planes%d", pl->tc_clen, pl->tc_nplanes);
  snprintf(in.variant_name, sizeof(in.variant_name), "tm_tc_bf16x3_hb%d_wc%d_seg%d_%s%s%s", tc::kHB, pl->tc_wc,
           pl->tc_nseg, mode_s, pl->tc_vcols ? "_cols" : "", roi ? "_roi" : "");
  fill_kernel_info(pl, (const void*)tm_tc_kernel, tc::kThreads, smem, nblk * pl->tc_vtiles * pl->tc_nseg, nsub, 1);
  in.specialized = 3;  // tensor-core tier: one kernel for every shape (h, w run-time evaluated), not an SK
  in.split = nblk;
  in.const_template = 0;
  in.slabs = 1;
  // template prep (+ operand), window sums, image split, numerator (+ chained block sum,
  // normalisation, argmax keys), tail (ragged columns' normalisation + peak), ragged columns
  in.launches_per_call = (h * w <= kPrepSmemFloats ? 1 : 2) + (pl->box_smem ? 1 : 2) + 3 + (pl->tc_vcols ? 1 : 0);
  return NCC_OK;
}

// Tiny problems (far below one wave): one launch does prep, window sums, numerator, normalise,
// argmax and the peak (tm_tiny_kernel), AOT-specialised for the template sizes below.  Taken when
// the band has at most kTinyOffsets offsets and a CTA's rows fit in shared memory; not for the
// generic / ROI / multi-template forms.  NCC_NO_TINY=1 keeps the general launch sequence.
constexpr int64_t kTinyOffsets = 16384;
ncc_status setup_tiny(ncc_plan pl) {
  const ncc_problem& p = pl->p;
  pl->tiny_fn = nullptr;
  const int h = p.tmpl_h, w = p.tmpl_w;
  const char* tc_env = getenv("NCC_TC");
  if ((p.flags & NCC_F_GENERIC_KERNEL) || pl->roi_mode || pl->n_tmpl != 1 || getenv("NCC_NO_TINY") ||
      (tc_env && atoi(tc_env) == 1) ||
      (int64_t)pl->Ub * pl->V > kTinyOffsets)
    return NCC_OK;
  const void* fn = nullptr;
  if (h == 16 && w == 16) fn = (const void*)tm_tiny_kernel<16, 16>;
  else if (h == 32 && w == 32) fn = (const void*)tm_tiny_kernel<32, 32>;
  if (!fn) return NCC_OK;
  // ~64 offsets per CTA (one per thread after the staging), at most one CTA per SM per frame
  int ctas = (int)std::min<int64_t>(ceil_div((int64_t)pl->Ub * pl->V, 64), pl->Ub);
  ctas = std::max(1, std::min(ctas, pl->nsm));
  const int rows = ceil_div(pl->Ub, ctas);
  ctas = ceil_div(pl->Ub, rows);
  const int64_t smem = (int64_t)rows * p.image_w * 16 + ((int64_t)h * w + (int64_t)(rows + h - 1) * p.image_w) * 4;
  if (smem > 96 * 1024) return NCC_OK;
  NCC_CUDA(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  ncc_status st;
  if ((st = dalloc(&pl->tiny_done, (size_t)p.batch))) return st;
  NCC_CUDA(cudaMemset(pl->tiny_done, 0, (size_t)p.batch * sizeof(unsigned int)));
  NCC_CUDA(cudaMemset(pl->keys, 0, (size_t)p.batch * sizeof(unsigned long long)));
  pl->tiny_fn = fn;
  pl->tiny_ctas = ctas;
  pl->tiny_rows = rows;
  pl->tiny_smem = (int)smem;
  ncc_plan_info& in = pl->info;
  snprintf(in.variant_name, sizeof(in.variant_name), "tm_tiny_%dx%d_c%d", h, w, ctas);
  fill_kernel_info(pl, fn, 256, (int)smem, ctas, p.batch, 1);
  in.specialized = 1;
  in.split = 1;
  in.const_template = 0;
  in.slabs = 1;
  in.launches_per_call = 1;
  return NCC_OK;
}

// SAD (ncc_sad.cuh): no numerator / window-sum decomposition; one direct kernel (+ key reset and
// peak).  Plain band matching only (no ROI / multi-template form).
ncc_status setup_sad_tm(ncc_plan pl, int maxsm) {
  const ncc_problem& p = pl->p;
  if (pl->roi_mode || pl->n_tmpl != 1) return NCC_ERR_UNSUPPORTED;
  const int w = p.tmpl_w;
  const int64_t smem = ((int64_t)kSadCH * w + (int64_t)(kSadCH + kSadTU - 1) * (kSadTV + w - 1 + 3)) * 4;
  if (smem > maxsm) return NCC_ERR_UNSUPPORTED;
  NCC_CUDA(cudaFuncSetAttribute((const void*)tm_sad_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  pl->sad = 1;
  pl->sad_smem = (int)smem;
  ncc_plan_info& in = pl->info;
  snprintf(in.variant_name, sizeof(in.variant_name), "tm_sad_%dx%d_rv%d", kSadTU, kSadTV, kSadRV);
  fill_kernel_info(pl, (const void*)tm_sad_kernel, 256, (int)smem, ceil_div(pl->V, kSadTV), ceil_div(pl->Ub, kSadTU),
                   p.batch);
  in.specialized = 0;
  in.variant_id = -1;
  in.split = 1;
  in.const_template = 0;
  in.slabs = 1;
  in.launches_per_call = 3;  // key reset, SAD, peak
  return NCC_OK;
}

ncc_status create_tm(ncc_plan pl) {
  const ncc_problem& p = pl->p;
  const int h = p.tmpl_h, w = p.tmpl_w;
  pl->U = p.image_h - h + 1;
  pl->V = p.image_w - w + 1;
  // balanced contiguous bands of offset rows: [r*U/n, (r+1)*U/n) (every band non-empty for n <= U)
  pl->u_begin = (int)((int64_t)p.shard_rank * pl->U / p.shard_count);
  pl->u_end = (int)((int64_t)(p.shard_rank + 1) * pl->U / p.shard_count);
  if (pl->u_begin >= pl->u_end) return NCC_ERR_INVALID_ARGUMENT;
  pl->Ub = pl->u_end - pl->u_begin;
  pl->Hs = pl->Ub + h - 1;
  pl->roi_mode = p.roi_h > 0;
  pl->n_tmpl = p.n_templates > 1 ? p.n_templates : 1;

  // variant selection (a8): AOT specialised instance > run-time specialised (NVRTC) > generic RE
  const TmVariant* v = &kTmVariants[0];
  bool aot = false;
  if (!(p.flags & NCC_F_GENERIC_KERNEL) && !tm_jit_forced(nullptr))
    for (const TmVariant& c : kTmVariants)
      if (c.TH == h && c.TW == w) {
        v = &c;
        aot = true;
        break;  // first matching specialised instance is the default
      }
  if (const char* force = getenv("NCC_FORCE_VARIANT"))  // sweeps: any instance valid for (h, w)
    for (const TmVariant& c : kTmVariants)
      if (strcmp(force, c.name) == 0 && (c.TH == 0 || (c.TH == h && c.TW == w))) {
        v = &c;
        aot = c.TH != 0;
      }
  if (!aot && jit_allowed(p.flags)) {
    TmJitChoice jc = tm_jit_choice(h, w);
    if (p.n_templates > 1) {  // several templates share the 64 KB constant bank or use shared memory
      const int64_t hp = ((h + jc.CH - 1) / jc.CH) * jc.CH, wp = ((w + jc.CW - 1) / jc.CW) * jc.CW;
      jc.ct = jc.ct && (int64_t)p.n_templates * hp * wp <= kConstTplFloats;
    }
    const std::vector<std::string> names = {tm_name(jc.RV, jc.LX, jc.WX, jc.WY, jc.CH, jc.CW, h, w, false, jc.ct),
                                            tm_name(jc.RV, jc.LX, jc.WX, jc.WY, jc.CH, jc.CW, h, w, true, jc.ct),
                                            "&nccb::c_tpl"};
    JitResult jr;
    std::string err;
    if (jit_build(names, &jr, &err) == NCC_OK) {
      NCC_CUDA(cudaLibraryLoadData(&pl->jit_lib, jr.cubin.data(), nullptr, nullptr, 0, nullptr, nullptr, 0));
      TmVariant jv = tm_geom(jc.RV, jc.LX, jc.WX, jc.WY, jc.CH, jc.CW);
      jv.TH = h;
      jv.TW = w;
      cudaKernel_t k0, k1;
      NCC_CUDA(cudaLibraryGetKernel(&k0, pl->jit_lib, jr.lowered[0].c_str()));
      NCC_CUDA(cudaLibraryGetKernel(&k1, pl->jit_lib, jr.lowered[1].c_str()));
      const int ct = jc.ct ? 1 : 0;
      pl->jit_ct = ct;
      jv.k[0][ct] = reinterpret_cast<const void*>(k0);
      jv.k[1][ct] = reinterpret_cast<const void*>(k1);
      jv.k[0][1 - ct] = jv.k[0][ct];  // only the chosen template source is compiled
      jv.k[1][1 - ct] = jv.k[1][ct];
      size_t csz = 0;
      NCC_CUDA(cudaLibraryGetGlobal(&pl->jit_ctpl, &csz, pl->jit_lib, jr.lowered[2].c_str()));
      pl->jit_ms = jr.cached ? 0.0 : jr.compile_ms;
      snprintf(pl->jit_name, sizeof(pl->jit_name), "tm_jit_%dx%d_rv%d_lx%d_%dx%d_c%dx%d%s", h, w, jc.RV, jc.LX, jc.WY,
               jc.WX, jc.CH, jc.CW, jr.cached ? "_cached" : "");
      jv.name = pl->jit_name;
      pl->tmv_store = jv;
      v = &pl->tmv_store;
    } else {
      g_last_cuda_error = err;  // reported via ncc_last_cuda_error; fall back to the generic kernel
    }
  }
  pl->tmv = v;
  const int nCH = ceil_div(h, v->CH), nCW = ceil_div(w, v->CW);
  pl->HP = nCH * v->CH;
  pl->WP = nCW * v->CW;

  int maxsm = 0, nsm = 0;
  NCC_CUDA(cudaDeviceGetAttribute(&maxsm, cudaDevAttrMaxSharedMemoryPerBlockOptin, pl->device));
  NCC_CUDA(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, pl->device));
  for (int t = 0; t < 2; ++t)
    for (int c = 0; c < 2; ++c) {
      if (pl->jit_lib && c != pl->jit_ct) continue;  // JIT: only the chosen template mode is compiled
      if (v->smem[t][c] > maxsm) return NCC_ERR_UNSUPPORTED;
      NCC_CUDA(cudaFuncSetAttribute(v->k[t][c], cudaFuncAttributeMaxDynamicSharedMemorySize, v->smem[t][c]));
    }
  const int rows_smem = (int)((kBoxRowsSEG + w + 1) * 2 * sizeof(double));
  if (rows_smem > maxsm) return NCC_ERR_UNSUPPORTED;
  NCC_CUDA(cudaFuncSetAttribute((const void*)box_rows_kernel<kBoxRowsNT>,
                                cudaFuncAttributeMaxDynamicSharedMemorySize, rows_smem));

  // constant-bank template: slabs of whole row-chunks that fit 64 KB (NCC_NO_CONST_TPL=1 disables)
  pl->slab_rows = (kConstTplFloats / pl->WP) / v->CH * v->CH;
  pl->use_ct = pl->jit_lib ? (pl->jit_ct != 0) : (pl->slab_rows >= v->CH && !getenv("NCC_NO_CONST_TPL"));
  if (pl->slab_rows > pl->HP) pl->slab_rows = pl->HP;
  pl->n_slabs = pl->use_ct ? ceil_div(pl->HP, pl->slab_rows) : 1;
  if (pl->n_tmpl > 1) {  // several templates: all of them resident in the constant bank, or shared memory
    const bool fits = (int64_t)pl->n_tmpl * pl->HP * pl->WP <= kConstTplFloats;
    pl->use_ct = pl->use_ct && fits;
    pl->slab_rows = pl->HP;
    pl->n_slabs = 1;
  }

  // tiles of this band; split-K factor S from the FULL problem's tile count (so every shard
  // of a problem uses the same S and the same per-offset accumulation order): the smallest
  // S <= chunks whose unit count fills whole "rounds" of resident CTAs to >= 97 %.
  pl->tiles_u = ceil_div(pl->roi_mode ? p.roi_h : pl->Ub, v->bu);
  pl->tiles_v = ceil_div(pl->roi_mode ? p.roi_w + 3 : pl->V, v->bv);  // ROI tiles start 16-B aligned
  {
    int per_sm = 0;
    const int ct = pl->use_ct ? 1 : 0;
    NCC_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, v->k[1][ct], v->nt, v->smem[1][ct]));
    const int64_t slots = (int64_t)(per_sm > 0 ? per_sm : 1) * nsm;
    const int64_t tiles_full = pl->roi_mode ? (int64_t)pl->tiles_u * pl->tiles_v * pl->n_tmpl
                                            : (int64_t)ceil_div(pl->U, v->bu) * ceil_div(pl->V, v->bv);
    const int nq = pl->n_slabs > 1 ? 1 : nCH * nCW;  // slab launches carry totals: no split
    // Equal-size units are scheduled dynamically; the tail is about half a unit's duration at
    // the per-SM concurrency, so aim for >= 6 "rounds" of resident units (measured on B200:
    // cfg2 54 -> 57 TFLOP/s from S = 4 to S = 8), then stop splitting.
    int best_s = 1;
    for (int S = 1; S <= nq && S <= 16; ++S) {
      best_s = S;
      if (tiles_full * S >= 6 * slots) break;
    }
    pl->split = best_s;
    if (const char* fs = getenv("NCC_FORCE_SPLIT")) {
      const int f = atoi(fs);
      if (f >= 1 && f <= nq) pl->split = f;
    }
  }

  NCC_CUDA(cudaStreamCreateWithFlags(&pl->side, cudaStreamNonBlocking));
  NCC_CUDA(cudaStreamCreateWithFlags(&pl->side2, cudaStreamNonBlocking));
  NCC_CUDA(cudaEventCreateWithFlags(&pl->ev_box, cudaEventDisableTiming));
  NCC_CUDA(cudaEventCreateWithFlags(&pl->ev_fork, cudaEventDisableTiming));
  NCC_CUDA(cudaEventCreateWithFlags(&pl->ev_join, cudaEventDisableTiming));
  NCC_CUDA(cudaEventCreateWithFlags(&pl->ev_cols, cudaEventDisableTiming));
  NCC_CUDA(cudaEventCreateWithFlags(&pl->ev_img, cudaEventDisableTiming));
  ncc_status st;
  if ((st = dalloc(&pl->tplC, (size_t)pl->n_tmpl * pl->HP * pl->WP))) return st;
  if ((st = dalloc(&pl->tst, (size_t)pl->n_tmpl))) return st;
  if ((st = dalloc(&pl->keys, (size_t)p.batch * pl->n_tmpl))) return st;
  const int64_t ntiles = (int64_t)pl->tiles_u * pl->tiles_v * p.batch * pl->n_tmpl;
  if (pl->split > 1) {
    if ((st = dalloc(&pl->part, (size_t)ntiles * pl->split * v->rv_nt()))) return st;
    if ((st = dalloc(&pl->cnt, (size_t)ntiles))) return st;
    NCC_CUDA(cudaMemset(pl->cnt, 0, (size_t)ntiles * sizeof(unsigned int)));
  }
  if (pl->n_slabs > 1)
    if ((st = dalloc(&pl->carry, (size_t)ntiles * v->rv_nt()))) return st;
  pl->rs_frame_stride = (int64_t)pl->Hs * pl->V;
  pl->s_frame_stride = (int64_t)pl->Ub * pl->V;
  if ((st = setup_box(pl, w))) return st;
  if (!pl->box_smem) {  // row-sum intermediate of the two-pass form only
    if ((st = dalloc(&pl->RS1, (size_t)p.batch * pl->rs_frame_stride))) return st;
    if ((st = dalloc(&pl->RS2, (size_t)p.batch * pl->rs_frame_stride))) return st;
  }
  if ((st = dalloc(&pl->S1, (size_t)p.batch * pl->s_frame_stride))) return st;
  if ((st = dalloc(&pl->S2, (size_t)p.batch * pl->s_frame_stride))) return st;
  {  // template chunks: 2D map over the zero-padded centred template
    const uint64_t dims[2] = {(uint64_t)pl->WP, (uint64_t)pl->HP * pl->n_tmpl};
    const uint64_t strides[1] = {(uint64_t)pl->WP * 4};
    const uint32_t box[2] = {(uint32_t)v->CW, (uint32_t)v->CH};
    pl->tma_ok = encode_f32(&pl->map_tpl, pl->tplC, 2, dims, strides, box);
  }

  ncc_plan_info& in = pl->info;
  in.U = pl->U;
  in.V = pl->V;
  in.u_begin = pl->u_begin;
  in.u_end = pl->u_end;
  in.outputs_per_call = pl->roi_mode ? (int64_t)p.roi_h * p.roi_w * p.batch * pl->n_tmpl
                                     : (int64_t)pl->Ub * pl->V * p.batch;
  in.flops_per_call = 2.0 * h * (double)w * (double)in.outputs_per_call;
  in.specialized = pl->jit_lib ? 2 : (v->TH != 0);
  in.variant_id = pl->jit_lib ? -1 : (int)(v - kTmVariants);
  snprintf(in.variant_name, sizeof(in.variant_name), "%s", v->name);
  snprintf(in.variant_name + strlen(in.variant_name), sizeof(in.variant_name) - strlen(in.variant_name), "_s%d%s",
           pl->split, pl->use_ct ? (pl->n_slabs > 1 ? "_cslab" : "_ctpl") : "_stpl");
  {
    const int ct = pl->use_ct ? 1 : 0;
    fill_kernel_info(pl, v->k[1][ct], v->nt, v->smem[1][ct], pl->tiles_u * pl->tiles_v * pl->split,
                     p.batch * pl->n_tmpl, 1);
    in.split = pl->split;
    in.const_template = pl->use_ct;
    in.slabs = pl->n_slabs;
    in.launches_per_call = 2 + (pl->box_smem ? 1 : 2) + pl->n_slabs;  // prep, window sums, numerator(s), finalize
  }
  if (p.score == NCC_SCORE_SAD) return setup_sad_tm(pl, maxsm);
  if ((st = setup_tiny(pl))) return st;
  if (pl->tiny_fn) return NCC_OK;
  return setup_tc(pl);
}

ncc_status create_piv(ncc_plan pl) {
  const ncc_problem& p = pl->p;
  const int h = p.tmpl_h, w = p.tmpl_w, my = p.search_y, mx = p.search_x;
  pl->Ky = (p.image_h - h - 2 * my) / p.step_y + 1;
  pl->Kx = (p.image_w - w - 2 * mx) / p.step_x + 1;
  pl->OY = 2 * my + 1;
  pl->OX = 2 * mx + 1;
  pl->map_h = p.image_h - h + 1;
  pl->map_w = p.image_w - w + 1;

  // variant selection (a8): AOT specialised instance > run-time specialised (NVRTC) > generic RE
  const PivVariant* v = &kPivVariants[0];
  bool aot = false;
  if (!(p.flags & NCC_F_GENERIC_KERNEL) && !getenv("NCC_PIV_JIT"))
    for (const PivVariant& c : kPivVariants)
      if (c.TH == h && c.TW == w && c.MY == my && c.MX == mx && !aot) {
        v = &c;  // first matching specialised instance is the default
        aot = true;
      }
  if (const char* force = getenv("NCC_FORCE_VARIANT"))  // sweeps: any instance valid for the shape
    for (const PivVariant& c : kPivVariants)
      if (strcmp(force, c.name) == 0 && (c.TH == 0 || (c.TH == h && c.TW == w && c.MY == my && c.MX == mx))) {
        v = &c;
        aot = c.TH != 0;
      }
  if (!aot && jit_allowed(p.flags)) {
    const PivJitChoice jc = piv_jit_choice(h, w, my, mx);
    if (jc.ok) {
      const std::vector<std::string> names = {
          piv_name(h, w, my, mx, jc.RV, jc.CW, jc.NT, jc.WPB, jc.MINB, true, true, 1),
          piv_name(h, w, my, mx, jc.RV, jc.CW, jc.NT, jc.WPB, jc.MINB, false, true, 1)};
      JitResult jr;
      std::string err;
      if (jit_build(names, &jr, &err) == NCC_OK) {
        NCC_CUDA(cudaLibraryLoadData(&pl->jit_lib, jr.cubin.data(), nullptr, nullptr, 0, nullptr, nullptr, 0));
        cudaKernel_t k0, k1;
        NCC_CUDA(cudaLibraryGetKernel(&k0, pl->jit_lib, jr.lowered[0].c_str()));
        NCC_CUDA(cudaLibraryGetKernel(&k1, pl->jit_lib, jr.lowered[1].c_str()));
        pl->jit_ms = jr.cached ? 0.0 : jr.compile_ms;
        snprintf(pl->jit_name, sizeof(pl->jit_name), "piv_jit_%dx%d_m%dx%d_rv%d_cw%d_nt%d_w%d%s", h, w, my, mx, jc.RV,
                 jc.CW, jc.NT, jc.WPB, jr.cached ? "_cached" : "");
        PivVariant jv{pl->jit_name, h, w, my, mx, jc.RV, jc.CW, jc.NT, jc.WPB, 1, 1,
                      reinterpret_cast<const void*>(k0), reinterpret_cast<const void*>(k1)};
        pl->pivv_store = jv;
        v = &pl->pivv_store;
      } else {
        g_last_cuda_error = err;
      }
    }
  }
  pl->pivv = v;
  const int RV = v->RV, CW = v->CW;
  const int NG = (pl->OX + RV - 1) / RV;
  pl->piv_bp = v->TH ? piv_sk_pitch(v->TW, v->MX, RV, CW) : piv_pick_pitch(NG * RV + ((w + CW - 1) / CW) * CW, RV, NG);
  (void)NG;
  const bool alias = v->ALIAS != 0;
  int items = 0;
  const PivShapeRT psr = piv_shape_rt(RV, CW, h, w, my, mx, pl->piv_bp, alias);
  const int64_t win_fl = psr.win_fl;
  items = psr.items;
  if (alias && (int64_t)items * v->WPB > (int64_t)v->NT * v->IPT) return NCC_ERR_UNSUPPORTED;
  pl->piv_smem = (int)(win_fl * 4 * v->WPB);
  int maxsm = 0;
  NCC_CUDA(cudaDeviceGetAttribute(&maxsm, cudaDevAttrMaxSharedMemoryPerBlockOptin, pl->device));
  if (win_fl * 4 * v->WPB > maxsm) return NCC_ERR_UNSUPPORTED;
  NCC_CUDA(cudaFuncSetAttribute(v->k_tma, cudaFuncAttributeMaxDynamicSharedMemorySize, pl->piv_smem));
  NCC_CUDA(cudaFuncSetAttribute(v->k_ldg, cudaFuncAttributeMaxDynamicSharedMemorySize, pl->piv_smem));
  if (v->k_ws && !getenv("NCC_NO_WS")) {  // persistent warp-specialised form: 2 stages + score tile
    PivShape<12, 64> ps(h, w, my, mx, pl->piv_bp, false);
    const int64_t ws_bytes = v->ws_bytes ? v->ws_bytes : (2 * (int64_t)(ps.tp_fl + ps.b_fl) + ps.s_fl) * 4;
    int nsm = 0;
    NCC_CUDA(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, pl->device));
    if (ws_bytes <= maxsm && (v->ws_bytes || (v->CW == 64 && v->RV == 12))) {
      pl->ws_bp = v->ws_bp ? v->ws_bp : pl->piv_bp;
      NCC_CUDA(cudaFuncSetAttribute(v->k_ws, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)ws_bytes));
      pl->ws_smem = (int)ws_bytes;
      pl->ws_grid = nsm;
    }
  }
  const int rows_smem = (int)((kBoxRowsSEG + w + 1) * 2 * sizeof(double));
  if (rows_smem > maxsm) return NCC_ERR_UNSUPPORTED;
  NCC_CUDA(cudaFuncSetAttribute((const void*)box_rows_kernel<kBoxRowsNT>,
                                cudaFuncAttributeMaxDynamicSharedMemorySize, rows_smem));

  // window-sum maps of frame B, processed in sub-batches of pairs
  pl->rs_frame_stride = (int64_t)p.image_h * pl->map_w;
  pl->s_frame_stride = (int64_t)pl->map_h * pl->map_w;
  ncc_status st;
  if ((st = setup_box(pl, w))) return st;
  // tensor-core numerator (f3 on the PIV path, ncc_piv_tc.cuh): NCC score, D_x = 2 m_x in {32, 64}
  // (R = 128 / D_x image rows per MMA), whole 16-column template chunks, and the overlapping windows
  // of a column strip fit the accumulator / operand slots.  NCC_PIV_TC=0 (or NCC_F_CUDA_CORES) keeps
  // the CUDA-core kernels.
  const char* e_ptc = getenv("NCC_PIV_TC");
  const int Dx = 2 * mx, R_ptc = (Dx == 32 || Dx == 64) ? 128 / Dx : 1, span_ptc = h + 2 * my;
  const bool ptc_ok = p.score == NCC_SCORE_NCC && !(p.flags & NCC_F_CUDA_CORES) && !(e_ptc && atoi(e_ptc) == 0) &&
                      (Dx == 32 || Dx == 64) && w % ptc::kKs == 0 && (h * w) % 128 == 0 &&
                      h * w <= 128 * ptc::kPrepMax && p.step_y % R_ptc == 0 && p.step_y <= span_ptc &&
                      (span_ptc + p.step_y - 1) / p.step_y <= ptc::kNSlot - 1 && p.step_x % 4 == 0 &&
                      p.image_pitch % 4 == 0 && Dx + w <= 256 && ptc::tmem_cols(my, R_ptc, w) <= 512 &&
                      ptc::smem_bytes(h, w, my, mx) <= maxsm && (2 * my + 1) * (2 * mx + 1) <= 128 * ptc::kEpiMax &&
                      2 * my + 1 <= 8 * kBorderDY;
  // default: the tensor cores where they measured faster (R = 2, +-32 search: cfg 4, 2.6x);
  // at R = 4 (+-16, cfg 3) the CUDA-core kernel wins (EXPERIMENTS.md); NCC_PIV_TC=1 forces them
  const bool use_ptc = ptc_ok && (R_ptc == 2 || (e_ptc && atoi(e_ptc) == 1));
  // Sub-batch sizing.  The CUDA-core kernels read fp64 window sums (16 B per map position, scratch
  // budget ~2 GiB); the tensor-core path reads only the fp32 factors (8 B) and its last-column
  // numerators, so its budget is 8 GiB -- cfg 4's 256 pairs in ONE sub-batch: the persistent
  // kernel's units (strips) then balance over the SMs to ~0.5 % instead of one partly filled wave
  // per 34-pair sub-batch (~7 %).  Sub-batches are equal-sized.  The host path streams chunks of
  // the 2 GiB size regardless (copy / compute overlap).
  const double per_pair_fp64 = 16.0 * (double)((pl->box_smem ? 0 : pl->rs_frame_stride) + pl->s_frame_stride);
  int sb_host = std::max(1, (int)(2.0 * 1024 * 1024 * 1024 / per_pair_fp64));
  int sb = sb_host;
  if (use_ptc && pl->box_smem) {
    const double per_pair = 8.0 * (double)pl->s_frame_stride + 4.0 * (double)pl->Ky * pl->Kx * pl->OY;
    sb = std::max(1, (int)(8.0 * 1024 * 1024 * 1024 / per_pair));
  }
  if (const char* e = getenv("NCC_PIV_SUB_BATCH")) {  // tests / sweeps
    sb = std::min(sb, std::max(1, atoi(e)));
    sb_host = std::min(sb_host, sb);
  }
  if (sb > p.batch) sb = p.batch;
  sb = ceil_div(p.batch, ceil_div(p.batch, sb));  // equal sub-batches
  pl->sub_batch = sb;
  pl->host_chunk = std::min(sb, std::min(sb_host, p.batch));
  if (!pl->box_smem) {
    if ((st = dalloc(&pl->RS1, (size_t)sb * pl->rs_frame_stride))) return st;
    if ((st = dalloc(&pl->RS2, (size_t)sb * pl->rs_frame_stride))) return st;
  }
  if (!(use_ptc && pl->box_smem)) {  // fp64 sums (the tensor-core path with the fused box kernel writes none)
    if ((st = dalloc(&pl->S1, (size_t)sb * pl->s_frame_stride))) return st;
    if ((st = dalloc(&pl->S2, (size_t)sb * pl->s_frame_stride))) return st;
  }
  {
    const int R = R_ptc, span = span_ptc;
    if (use_ptc) {
      pl->ptc = 1;
      pl->ptc_R = R;
      pl->ptc_smem = ptc::smem_bytes(h, w, my, mx);
      pl->ptc_border_smem = (h * w + (span + kBorderDY - 1) * w) * 4;
      // register-blocked last-column kernel for 32- / 64-row masks of 32 / 64 columns
      pl->ptc_border_rb = ((h == 32 || h == 64) && (w == 32 || w == 64) && !getenv("NCC_PIV_TC_BORDER_GENERIC")) ? h : 0;
      if (pl->ptc_border_rb) {
        pl->ptc_border_smem += 8 * (w / 32) * kBorderDY * 4;
        const void* f = pl->ptc_border_rb == 64 ? (const void*)piv_tc_border_rb<64> : (const void*)piv_tc_border_rb<32>;
        NCC_CUDA(cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, pl->ptc_border_smem));
      }
      if (pl->ptc_border_smem > maxsm) return NCC_ERR_UNSUPPORTED;
      NCC_CUDA(cudaFuncSetAttribute((const void*)piv_tc_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, pl->ptc_smem));
      NCC_CUDA(cudaFuncSetAttribute((const void*)piv_tc_border_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                    pl->ptc_border_smem));
      if ((st = dalloc(&pl->ptc_border, (size_t)sb * pl->Ky * pl->Kx * pl->OY))) return st;
      if (getenv("NCC_PIV_TC_PROF")) {
        if ((st = dalloc(&pl->ptc_prof, (size_t)pl->nsm * 32 + 3 * 2048))) return st;
        NCC_CUDA(cudaMemset(pl->ptc_prof, 0, ((size_t)pl->nsm * 32 + 3 * 2048) * 8));
      }
    }
  }
  if (p.score == NCC_SCORE_NCC && (pl->ws_smem || pl->ptc)) {  // fp32 normalisation factors (WS / TC kernels)
    if ((st = dalloc(&pl->tc_rsv, (size_t)sb * pl->s_frame_stride))) return st;
    if ((st = dalloc(&pl->tc_mean, (size_t)sb * pl->s_frame_stride))) return st;
  }

  ncc_plan_info& in = pl->info;
  in.U = pl->OY;
  in.V = pl->OX;
  in.Ky = pl->Ky;
  in.Kx = pl->Kx;
  in.outputs_per_call = (int64_t)pl->Ky * pl->Kx * p.batch;
  in.flops_per_call = 2.0 * h * (double)w * pl->OY * (double)pl->OX * (double)in.outputs_per_call;
  in.specialized = pl->jit_lib ? 2 : (v->TH != 0);
  in.variant_id = pl->jit_lib ? -1 : (int)(v - kPivVariants);
  snprintf(in.variant_name, sizeof(in.variant_name), "%s", v->name);
  if (pl->ws_smem)  // persistent warp-specialised kernel: one CTA per SM loops over the windows
    fill_kernel_info(pl, v->k_ws, (v->ws_ncw + v->ws_npw) * 32, pl->ws_smem, pl->ws_grid, 1, sb);  // z: pairs per launch
  else
    fill_kernel_info(pl, v->k_ldg, v->NT, pl->piv_smem, ceil_div((int64_t)pl->Ky * pl->Kx, v->WPB), 1, sb);
  in.launches_per_call = (pl->box_smem ? 2 : 3) * ceil_div(p.batch, sb);  // per sub-batch: window sums + PIV
  if (pl->ptc) {  // per sub-batch: window sums, last-column kernel, tensor-core kernel
    int nsm = 0;
    NCC_CUDA(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, pl->device));
    snprintf(in.variant_name, sizeof(in.variant_name), "piv_tc_bf16x3_%dx%d_m%dx%d_r%d", h, w, my, mx, pl->ptc_R);
    fill_kernel_info(pl, (const void*)piv_tc_kernel, ptc::kThreads, pl->ptc_smem, nsm, 1, 1);
    in.specialized = 3;
    in.variant_id = -1;
    in.launches_per_call = (pl->box_smem ? 3 : 4) * ceil_div(p.batch, sb);
  }
  if (p.score == NCC_SCORE_SAD) {  // direct |t - b| kernel, one CTA per (window, pair); no window sums
    const int OY = 2 * my + 1, OX = 2 * mx + 1, OXP = ((OX + 3) / 4) * 4;
    const int64_t smem = ((int64_t)h * w + (int64_t)(h + 2 * my) * (w + 2 * mx + 3) + (int64_t)OY * OXP) * 4;
    if (smem > maxsm) return NCC_ERR_UNSUPPORTED;
    NCC_CUDA(cudaFuncSetAttribute((const void*)piv_sad_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    pl->sad = 1;
    pl->sad_smem = (int)smem;
    snprintf(in.variant_name, sizeof(in.variant_name), "piv_sad_%dx%d_m%dx%d", h, w, my, mx);
    fill_kernel_info(pl, (const void*)piv_sad_kernel, 256, (int)smem, pl->Ky * pl->Kx, sb, 1);
    in.specialized = 0;
    in.variant_id = -1;
    in.launches_per_call = ceil_div(p.batch, sb);
  }
  return NCC_OK;
}

ncc_status ensure_events(ncc_plan pl, int n) {
  while ((int)pl->ev.size() < n) {
    cudaEvent_t e;
    NCC_CUDA(cudaEventCreate(&e));
    pl->ev.push_back(e);
  }
  return NCC_OK;
}

inline void mark(ncc_plan pl, cudaStream_t s, int i) {
  // under graph capture an event record is a dependency marker unless recorded as external:
  // then it becomes an event-record node that the replay executes (timing stays valid)
  if (pl->p.flags & NCC_F_TIMING) cudaEventRecordWithFlags(pl->ev[i], s, pl->capturing ? cudaEventRecordExternal : 0);
}

// window sums of `batch` frames over rows [row0, row0 + rows_out + h - 1)
// pdl: launched as a programmatic dependent of the preceding kernel in `s` (the tensor-core
// numerator, which triggers it at its start): the window sums then run on the SMs the numerator
// leaves free, instead of in front of it.
void launch_box(ncc_plan pl, const float* frames, int batch, int row0, int rows_out, cudaStream_t s, bool pdl = false,
                bool factors_only = false) {
  const ncc_problem& p = pl->p;
  // factors_only: the tensor-core NCC path reads only the fp32 factors (rsqrt(n var), S1/n), not
  // the fp64 sums (12.9 MB of stores at cfg 2)
  double* const S1o = factors_only && pl->box_smem ? nullptr : pl->S1;
  double* const S2o = factors_only && pl->box_smem ? nullptr : pl->S2;
  const int h = p.tmpl_h, w = p.tmpl_w;
  const int V = p.image_w - w + 1;
  if (pl->box_smem) {  // fused single pass; rows per CTA halved until the grid covers every SM
    const int gx = ceil_div(V, kBoxTV);
    int TU = 64;
    while (TU > pl->box_r && (int64_t)gx * ceil_div(rows_out, TU) * batch < pl->nsm) TU /= 2;
    if (const char* e = getenv("NCC_BOX_TU")) TU = std::max(pl->box_r, atoi(e));  // sweeps
    dim3 g(gx, ceil_div(rows_out, TU), batch);
    if (pdl) {
      cudaLaunchConfig_t cfg = {};
      cfg.gridDim = g;
      cfg.blockDim = dim3(kBox2dNT);
      cfg.dynamicSmemBytes = (size_t)pl->box_smem;
      cfg.stream = s;
      cudaLaunchAttribute at[1];
      at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
      at[0].val.programmaticStreamSerializationAllowed = 1;
      cfg.attrs = at;
      cfg.numAttrs = 1;
      const int64_t fs = (int64_t)p.image_h * p.image_pitch, sfs = pl->s_frame_stride;
      const int tv = kBoxTV;
      cudaLaunchKernelEx(&cfg, box2d_kernel<kBox2dNT>, frames, p.image_pitch, fs, row0, h, w, V, rows_out, tv, TU,
                         pl->box_r, pl->box_iwp, S1o, S2o, sfs, pl->tc_rsv, pl->tc_mean,
                         1.0 / ((double)h * (double)w));
      return;
    }
    box2d_kernel<kBox2dNT><<<g, kBox2dNT, pl->box_smem, s>>>(frames, p.image_pitch,
                                                            (int64_t)p.image_h * p.image_pitch, row0, h, w, V,
                                                            rows_out, kBoxTV, TU, pl->box_r, pl->box_iwp, S1o,
                                                            S2o, pl->s_frame_stride, pl->tc_rsv, pl->tc_mean,
                                                            1.0 / ((double)h * (double)w));
    return;
  }
  const int rows_in = rows_out + h - 1;
  const int seg = V < kBoxRowsSEG ? V : kBoxRowsSEG;
  const int smem = (int)((seg + w + 1) * 2 * sizeof(double));
  dim3 g1(ceil_div(V, seg), rows_in, batch);
  box_rows_kernel<kBoxRowsNT><<<g1, kBoxRowsNT, smem, s>>>(frames, p.image_pitch, (int64_t)p.image_h * p.image_pitch,
                                                           p.image_w, row0, w, V, seg, pl->RS1, pl->RS2,
                                                           pl->rs_frame_stride);
  dim3 g2(ceil_div(V, 32), ceil_div(rows_out, kBoxColsNW * kBoxColsL), batch);
  box_cols_kernel<kBoxColsNW, kBoxColsL><<<g2, kBoxColsNW * 32, 0, s>>>(pl->RS1, pl->RS2, pl->rs_frame_stride, V, h,
                                                                        rows_out, pl->S1, pl->S2, pl->s_frame_stride, pl->tc_rsv, pl->tc_mean, 1.0 / ((double)h * (double)w));
}

bool getenv_flag_two_kernel_prep() {  // NCC_TC_TWO_KERNEL_PREP=1: the earlier two-launch template prep
  static const bool v = getenv("NCC_TC_TWO_KERNEL_PREP") != nullptr;
  return v;
}

// `nframes` frames (<= the plan's batch; -1 = all) from d_images; peaks / surfaces of frame k at
// index k (the host path streams chunks of frames through this).
ncc_status run_match(ncc_plan pl, const float* d_images, const float* d_tmpl, int64_t tmpl_pitch, float* d_scores,
                     ncc_peak* d_peaks, cudaStream_t s, const int32_t* d_rois = nullptr, int nframes = -1) {
  const ncc_problem& p = pl->p;
  const int batch = nframes < 0 ? p.batch : nframes;
  const TmVariant* v = pl->tmv;
  if (p.flags & NCC_F_TIMING) {
    ncc_status st = ensure_events(pl, 5);
    if (st) return st;
  }
  pl->timing_kind = 1;
  if (pl->sad) {  // SAD: key reset, the direct kernel, peak (argmin)
    mark(pl, s, 0);
    if (pl->h_tmpl_in) {
      NCC_CUDA(cudaMemcpy2DAsync(const_cast<float*>(d_tmpl), tmpl_pitch * sizeof(float), pl->h_tmpl_in,
                                 pl->h_tmpl_pitch * sizeof(float), p.tmpl_w * sizeof(float), p.tmpl_h,
                                 cudaMemcpyHostToDevice, s));
      NCC_CUDA(cudaMemcpyAsync(const_cast<float*>(d_images), pl->h_img_in,
                               (size_t)batch * p.image_h * p.image_pitch * sizeof(float), cudaMemcpyHostToDevice, s));
    }
    tm_keys_reset<<<ceil_div(batch, 128), 128, 0, s>>>(pl->keys, batch);
    mark(pl, s, 1);
    mark(pl, s, 2);
    tm_sad_kernel<<<dim3(ceil_div(pl->V, kSadTV), ceil_div(pl->Ub, kSadTU), batch), 256, pl->sad_smem, s>>>(
        d_images, p.image_pitch, (int64_t)p.image_h * p.image_pitch, p.image_h, p.image_w, d_tmpl, tmpl_pitch,
        p.tmpl_h, p.tmpl_w, pl->u_begin, pl->Ub, pl->V, (p.flags & NCC_F_WRITE_SURFACE) ? d_scores : nullptr,
        (int64_t)pl->Ub * pl->V, pl->keys);
    mark(pl, s, 3);
    tm_finalize<<<ceil_div(batch, 128), 128, 0, s>>>(pl->keys, pl->tst, pl->V, reinterpret_cast<PeakOut*>(d_peaks),
                                                     batch, 1, 1);
    mark(pl, s, 4);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(e, "ncc_match launch (SAD)");
    return NCC_OK;
  }
  if (pl->tiny_fn) {  // the whole path in one launch
    mark(pl, s, 0);
    if (pl->h_tmpl_in) {
      NCC_CUDA(cudaMemcpy2DAsync(const_cast<float*>(d_tmpl), tmpl_pitch * sizeof(float), pl->h_tmpl_in,
                                 pl->h_tmpl_pitch * sizeof(float), p.tmpl_w * sizeof(float), p.tmpl_h,
                                 cudaMemcpyHostToDevice, s));
      NCC_CUDA(cudaMemcpyAsync(const_cast<float*>(d_images), pl->h_img_in,
                               (size_t)batch * p.image_h * p.image_pitch * sizeof(float), cudaMemcpyHostToDevice, s));
    }
    mark(pl, s, 1);
    mark(pl, s, 2);
    float* scores = (p.flags & NCC_F_WRITE_SURFACE) ? d_scores : nullptr;
    int64_t fs = (int64_t)p.image_h * p.image_pitch, sfs = (int64_t)pl->Ub * pl->V;
    int W = p.image_w, h = p.tmpl_h, w = p.tmpl_w, ub = pl->u_begin, Ubv = pl->Ub, V = pl->V, rows = pl->tiny_rows;
    int ssd = p.score == NCC_SCORE_SSD;
    int64_t pitch = p.image_pitch;
    void* args[] = {&d_images, &pitch, &fs, &W, &d_tmpl, &tmpl_pitch, &h, &w, &ub, &Ubv, &V, &rows,
                    &scores, &sfs, &pl->keys, &pl->tiny_done, &d_peaks, &ssd};
    NCC_CUDA(cudaLaunchKernel(pl->tiny_fn, dim3(pl->tiny_ctas, batch), dim3(256), args, (size_t)pl->tiny_smem, s));
    mark(pl, s, 3);
    mark(pl, s, 4);
    return NCC_OK;
  }
  CUtensorMap map_tc;
  bool tc_now = false;
  if (pl->tc) {  // the band's image operand (tm_tc_split): wp x 2 planes x Hs x batch 8-byte elements
    const int wp = (p.image_w + 1) & ~1;  // elements per plane row (16-byte TMA strides)
    const uint64_t dims[4] = {(uint64_t)wp, 2u, (uint64_t)pl->Hs, (uint64_t)batch};
    const uint64_t strides[3] = {(uint64_t)wp * 8, (uint64_t)wp * 16, (uint64_t)pl->Hs * wp * 16};
    const uint32_t box[4] = {(uint32_t)tc::kBoxW, 2u, 1u, 1u};
    tc_now = encode_f32(&map_tc, pl->tc_img2, 4, dims, strides, box, true);
  }
  const int nblk_tc = pl->tc_nbi * pl->tc_nbj;
  const bool tc_factors_only = tc_now && p.score == NCC_SCORE_NCC;  // no fp64 window-sum stores needed
  auto launch_cols = [&]() {  // the ragged last columns (tensor-core path), on the side stream
    if (pl->h_img_in) cudaStreamWaitEvent(pl->side, pl->ev_img, 0);  // host path: frames copied (errors: cudaGetLastError below)
    // small templates: one output per warp (short CTAs that finish before the tensor-core grid
    // needs their SMs, cfg 2); large ones: 4 sliding rows per warp (a quarter of the loads;
    // cfg 5: 740 -> 329 us, no longer delaying the numerator's start)
    constexpr int RWN = 4;
    const int jc = ceil_div(p.tmpl_w, 32);
    const int64_t items = (int64_t)batch * (jc <= 8 ? pl->Ub : ceil_div(pl->Ub, RWN)) * pl->tc_vcols;
    const int64_t pfs = (int64_t)pl->Ub * pl->V;
    auto cols = [&](auto kern) {
      kern<<<(unsigned)ceil_div(items, 8), 256, 0, pl->side>>>(
          d_images, p.image_pitch, (int64_t)p.image_h * p.image_pitch, pl->tplC, pl->WP, p.tmpl_h, p.tmpl_w,
          pl->V - pl->tc_vcols, pl->V, pl->u_begin, pl->Ub, batch, pl->tc_planes ? pl->tc_part : pl->tc_acc, pfs);
    };
    if (jc <= 4) cols(tm_tc_cols<4>);
    else if (jc <= 8) cols(tm_tc_cols<8>);
    else cols(tm_tc_cols_rw<16, RWN>);
  };
  auto launch_split = [&](cudaStream_t st) {
    const int wp = (p.image_w + 1) & ~1;
    tm_tc_split<<<dim3(ceil_div(ceil_div(wp, 4), 128), pl->Hs, batch), 128, 0, st>>>(
        d_images, p.image_pitch, (int64_t)p.image_h * p.image_pitch, p.image_w, pl->u_begin,
        reinterpret_cast<uint2*>(pl->tc_img2), (int64_t)pl->Hs * 2 * wp, wp,
        pl->tc_center ? pl->tst : nullptr, (double)p.tmpl_h * p.tmpl_w);
  };
  // fork: template prep on the side stream.  Host path: the template's copy (small) goes first,
  // then the frames' copy on the main stream runs beside the template prep; the side stream's
  // only reader of the frames (the ragged-column kernel) waits for the frames' copy (ev_img) --
  // the main stream's kernels are ordered after it anyway.
  mark(pl, s, 0);
  if (pl->h_tmpl_in)  // small: first on the copy engine, so the prep overlaps the frames' copy
    NCC_CUDA(cudaMemcpy2DAsync(const_cast<float*>(d_tmpl), tmpl_pitch * sizeof(float), pl->h_tmpl_in,
                               pl->h_tmpl_pitch * sizeof(float), p.tmpl_w * sizeof(float), p.tmpl_h,
                               cudaMemcpyHostToDevice, s));
  NCC_CUDA(cudaEventRecord(pl->ev_fork, s));
  NCC_CUDA(cudaStreamWaitEvent(pl->side, pl->ev_fork, 0));
  if (pl->h_img_in) {
    NCC_CUDA(cudaMemcpyAsync(const_cast<float*>(d_images), pl->h_img_in,
                             (size_t)batch * p.image_h * p.image_pitch * sizeof(float), cudaMemcpyHostToDevice, s));
    NCC_CUDA(cudaEventRecord(pl->ev_img, s));
  }
  if (pl->tc && p.tmpl_h * p.tmpl_w <= kPrepSmemFloats && !getenv_flag_two_kernel_prep()) {
    // one launch: template stats + centred template + MMA operand, template staged in shared memory
    tm_tc_prep<<<dim3(nblk_tc, pl->n_tmpl), 1024, p.tmpl_h * p.tmpl_w * 4, pl->side>>>(d_tmpl, tmpl_pitch, p.tmpl_h, p.tmpl_w, pl->tplC, pl->HP, pl->WP,
                                               pl->tst, pl->keys, batch, pl->tc_wc, pl->tc_nbj, pl->tcB);
    mark(pl, pl->side, 1);
  } else {
    tm_template_prep<<<pl->n_tmpl, 1024, 0, pl->side>>>(d_tmpl, tmpl_pitch, p.tmpl_h, p.tmpl_w, pl->tplC, pl->HP,
                                                         pl->WP, pl->tst, pl->keys, batch);
    mark(pl, pl->side, 1);
    if (pl->tc)
      tm_tc_tpl_prep<<<nblk_tc, 256, 0, pl->side>>>(pl->tplC, pl->WP, p.tmpl_h, p.tmpl_w, pl->tc_wc, pl->tc_nbj,
                                                    pl->tcB);
  }
  // the image split on the side stream after the template prep: for the centred operand (it needs
  // the template mean), and in schedule 4 (window sums first on the main stream, alone)
  const bool split_side = tc_now && (pl->tc_center || pl->tc_sched == 4);
  if (split_side) {
    if (pl->h_img_in) NCC_CUDA(cudaStreamWaitEvent(pl->side, pl->ev_img, 0));
    launch_split(pl->side);
  }
  NCC_CUDA(cudaEventRecord(pl->ev_join, pl->side));
  const bool box_beside = tc_now && pl->tc_sched == 5 && pl->tc_planes;
  if (box_beside) {
    // planes mode: the numerator does not read the window sums (tm_tc_finish does), so they run on
    // a second side stream from the start, beside the template prep and the image split; the
    // numerator waits only for those two and starts on the SMs the window sums leave free
    NCC_CUDA(cudaStreamWaitEvent(pl->side2, pl->ev_fork, 0));
    if (pl->h_img_in) NCC_CUDA(cudaStreamWaitEvent(pl->side2, pl->ev_img, 0));
    launch_box(pl, d_images, batch, pl->u_begin, pl->Ub, pl->side2, false, tc_factors_only);
    NCC_CUDA(cudaEventRecord(pl->ev_box, pl->side2));
    if (pl->tc_vcols) {
      launch_cols();
      NCC_CUDA(cudaEventRecord(pl->ev_cols, pl->side));
    }
    if (!split_side) launch_split(s);
    NCC_CUDA(cudaStreamWaitEvent(s, pl->ev_join, 0));
    mark(pl, s, 2);
  } else if (tc_now && pl->tc_sched == 4) {
    // window sums first, alone on the main stream (232 CTAs at 2 per SM leave room for the
    // template prep's few CTAs); prep -> image split -> ragged columns on the side stream
    if (pl->tc_vcols) {
      launch_cols();
      NCC_CUDA(cudaEventRecord(pl->ev_cols, pl->side));
    }
    launch_box(pl, d_images, batch, pl->u_begin, pl->Ub, s, false, tc_factors_only);
    NCC_CUDA(cudaStreamWaitEvent(s, pl->ev_join, 0));
    mark(pl, s, 2);
  } else if (tc_now && (pl->tc_sched == 3 || pl->tc_sched == 6)) {
    // the image split first (small: it leaves room for the template prep, which starts at once
    // on the side stream), then the window sums on the main stream; the ragged columns follow
    // the template prep on the side stream and overlap the window sums / tensor-core kernel
    if (pl->tc_vcols) {
      launch_cols();
      NCC_CUDA(cudaEventRecord(pl->ev_cols, pl->side));
    }
    if (pl->tc_sched == 6) {
      // schedule 6: the window sums on a second side stream from the start, beside the image split
      // (neither reads the other's output); the numerator waits for both
      NCC_CUDA(cudaStreamWaitEvent(pl->side2, pl->ev_fork, 0));
      if (pl->h_img_in) NCC_CUDA(cudaStreamWaitEvent(pl->side2, pl->ev_img, 0));
      launch_box(pl, d_images, batch, pl->u_begin, pl->Ub, pl->side2, false, tc_factors_only);
      NCC_CUDA(cudaEventRecord(pl->ev_box, pl->side2));
    }
    if (!split_side) launch_split(s);
    // planes mode: the numerator does not read the window sums (tm_tc_finish does), so they run
    // after it as its programmatic dependent, on the SMs it leaves free (cfg2: 8 of 148)
    if (pl->tc_sched == 6)
      NCC_CUDA(cudaStreamWaitEvent(s, pl->ev_box, 0));
    else if (!(pl->tc_planes && pl->box_smem && pl->tc_box_late))
      launch_box(pl, d_images, batch, pl->u_begin, pl->Ub, s, false, tc_factors_only);
    NCC_CUDA(cudaStreamWaitEvent(s, pl->ev_join, 0));
    mark(pl, s, 2);
  } else {
    // window sums on the main stream while the template prep runs on the side stream (the
    // tensor-core kernel normalises in its drains, so the window sums always precede it)
    if (tc_now && pl->tc_vcols) {  // after the join: overlaps the tensor-core kernel rather than delay its start
      launch_cols();
      NCC_CUDA(cudaEventRecord(pl->ev_cols, pl->side));
    }
    launch_box(pl, d_images, batch, pl->u_begin, pl->Ub, s, false, tc_factors_only);
    NCC_CUDA(cudaStreamWaitEvent(s, pl->ev_join, 0));
    mark(pl, s, 2);
  }
  if (tc_now) {  // tensor-core numerator, then block sum + normalisation + argmax
    const int nblk = nblk_tc;
    if (!split_side && !box_beside && pl->tc_sched != 3 && pl->tc_sched != 6) launch_split(s);  // schedules 0 / 5-chain
    TcArgs t;
    t.H = p.image_h;
    t.W = p.image_w;
    t.tcB = pl->tcB;
    t.WC = pl->tc_wc;
    t.nbi = pl->tc_nbi;
    t.nbj = pl->tc_nbj;
    t.V = pl->V;
    t.u_begin = pl->u_begin;
    t.u_end = pl->u_end;
    t.useg = pl->tc_useg;
    t.nseg = pl->tc_nseg;
    t.vtiles = pl->tc_vtiles;
    t.acc = pl->tc_acc;
    t.planes = pl->tc_planes;
    t.clen = pl->tc_clen;
    t.acc_chain_stride = (int64_t)p.batch * pl->Ub * pl->V;
    t.rois = pl->roi_mode ? d_rois : nullptr;
    t.n_tmpl = pl->n_tmpl;
    t.roi_h = p.roi_h;
    t.roi_w = p.roi_w;
    t.U = pl->U;
    t.part = pl->tc_part;
    t.part_blk_stride = pl->roi_mode ? (int64_t)p.batch * pl->n_tmpl * p.roi_h * p.roi_w
                                     : (int64_t)p.batch * pl->Ub * pl->V;
    t.acc_frame_stride = (int64_t)pl->Ub * pl->V;
    t.flags = pl->tc_flags;
    t.ngrp_max = pl->tc_ngrp;
    t.ticket = pl->tc_ticket;
    t.S1 = pl->S1;
    t.S2 = pl->S2;
    t.rsv = pl->tc_rsv;
    t.mean = pl->tc_mean;
    t.stat_frame_stride = pl->s_frame_stride;
    t.tst = pl->tst;
    t.h = p.tmpl_h;
    t.w = p.tmpl_w;
    t.scores = (p.flags & NCC_F_WRITE_SURFACE) ? d_scores : nullptr;
    t.score_frame_stride = (int64_t)pl->Ub * pl->V;
    t.keys = pl->keys;
    t.ssd = p.score == NCC_SCORE_SSD;
    t.exp = pl->tc_exp;
    t.prof = pl->tc_prof;
    t.center = pl->tc_center;
    tm_tc_kernel<<<dim3(nblk * pl->tc_vtiles * pl->tc_nseg, batch * pl->n_tmpl), tc::kThreads,
                   tc::smem_bytes(pl->tc_wc), s>>>(
        t, map_tc);
    if (pl->tc_sched == 3 && pl->tc_planes && pl->box_smem && pl->tc_box_late)
      launch_box(pl, d_images, batch, pl->u_begin, pl->Ub, s, /*pdl=*/true, tc_factors_only);
    mark(pl, s, 3);
    if (pl->tc_vcols) NCC_CUDA(cudaStreamWaitEvent(s, pl->ev_cols, 0));
    if (box_beside) NCC_CUDA(cudaStreamWaitEvent(s, pl->ev_box, 0));
    if (pl->roi_mode) {
      const int nsub = batch * pl->n_tmpl;
      tm_tc_finish_roi<<<dim3(ceil_div(p.roi_w, 256 * kFinV), p.roi_h, nsub), 256, 0, s>>>(
          pl->tc_part, nblk, (int64_t)p.batch * pl->n_tmpl * p.roi_h * p.roi_w, d_rois, pl->n_tmpl, p.roi_h, p.roi_w,
          pl->U, pl->V, pl->tc_rsv, pl->tc_mean, pl->S1, pl->S2, pl->s_frame_stride, pl->tst, p.tmpl_h, p.tmpl_w,
          (p.flags & NCC_F_WRITE_SURFACE) ? d_scores : nullptr, pl->keys, p.score == NCC_SCORE_SSD, pl->tc_done,
          reinterpret_cast<PeakOut*>(d_peaks), nsub);
    } else if (pl->tc_planes) {
      tm_tc_finish<<<dim3(ceil_div(pl->V, 256 * kFinV), ceil_div(pl->Ub, kFinR), batch), 256, 0, s>>>(
          pl->tc_part, pl->tc_nplanes, (int64_t)p.batch * pl->Ub * pl->V, (int64_t)pl->Ub * pl->V, pl->tc_rsv, pl->tc_mean,
          pl->S1, pl->S2, pl->s_frame_stride, pl->tst, p.tmpl_h, p.tmpl_w, pl->V, pl->V - pl->tc_vcols, pl->u_begin,
          (p.flags & NCC_F_WRITE_SURFACE) ? d_scores : nullptr, (int64_t)pl->Ub * pl->V, pl->keys,
          p.score == NCC_SCORE_SSD, pl->tc_done, reinterpret_cast<PeakOut*>(d_peaks), batch, pl->Ub);
    } else {
      const int64_t tail_items = (int64_t)batch * pl->Ub * pl->tc_vcols;
      tm_tc_tail<<<(unsigned)std::max<int64_t>(1, ceil_div(tail_items, 256)), 256, 0, s>>>(
          pl->tc_acc, (int64_t)pl->Ub * pl->V, pl->tc_rsv, pl->tc_mean, pl->S1, pl->S2, pl->s_frame_stride, pl->tst, p.tmpl_h, p.tmpl_w, pl->V,
          pl->V - pl->tc_vcols, pl->u_begin, pl->Ub, batch, (p.flags & NCC_F_WRITE_SURFACE) ? d_scores : nullptr,
          (int64_t)pl->Ub * pl->V, pl->keys, p.score == NCC_SCORE_SSD, pl->tc_done, reinterpret_cast<PeakOut*>(d_peaks));
    }
    mark(pl, s, 4);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(e, "ncc_match launch (tensor core)");
    return NCC_OK;
  }
  TmArgs a;
  a.img = d_images;
  a.pitch = p.image_pitch;
  a.frame_stride = (int64_t)p.image_h * p.image_pitch;
  a.H = p.image_h;
  a.W = p.image_w;
  a.tplC = pl->tplC;
  a.tplP = pl->WP;
  a.h = p.tmpl_h;
  a.w = p.tmpl_w;
  a.nCH = pl->HP / v->CH;
  a.nCW = pl->WP / v->CW;
  a.S1 = pl->S1;
  a.S2 = pl->S2;
  a.stat_frame_stride = pl->s_frame_stride;
  a.tst = pl->tst;
  a.U = pl->U;
  a.V = pl->V;
  a.u_begin = pl->u_begin;
  a.u_end = pl->u_end;
  a.tiles_u = pl->tiles_u;
  a.tiles_v = pl->tiles_v;
  a.scores = (p.flags & NCC_F_WRITE_SURFACE) ? d_scores : nullptr;
  a.score_frame_stride = (int64_t)pl->Ub * pl->V;
  a.keys = pl->keys;
  a.part = pl->part;
  a.cnt = pl->cnt;
  a.S = pl->split;
  a.ssd = p.score == NCC_SCORE_SSD;
  a.n_tmpl = pl->n_tmpl;
  a.roi = pl->roi_mode ? d_rois : nullptr;
  a.roi_h = p.roi_h;
  a.roi_w = p.roi_w;
  a.tpl_stride = (int64_t)pl->HP * pl->WP;
  a.tpl_rows = pl->HP;
  a.map_u0 = pl->u_begin;
  // TMA needs a 16-B aligned base and a pitch that is a multiple of 16 B; else plain loads.
  CUtensorMap map_img;
  memset(&map_img, 0, sizeof(map_img));
  bool use_tma = pl->tma_ok && (reinterpret_cast<uintptr_t>(d_images) % 16 == 0) && (p.image_pitch % 4 == 0);
  if (use_tma) {
    const uint64_t dims[3] = {(uint64_t)p.image_w, (uint64_t)p.image_h, (uint64_t)batch};
    const uint64_t strides[2] = {(uint64_t)p.image_pitch * 4, (uint64_t)p.image_h * p.image_pitch * 4};
    const uint32_t box[3] = {(uint32_t)v->ip, (uint32_t)v->ir, 1u};
    use_tma = encode_f32(&map_img, d_images, 3, dims, strides, box);
  }
  dim3 grid(pl->tiles_u * pl->tiles_v * pl->split, batch * pl->n_tmpl);
  const int t = use_tma ? 1 : 0, ct = pl->use_ct ? 1 : 0;
  const int nCWl = pl->WP / v->CW;
  a.carry = pl->carry;
  void* args[3] = {&a, &map_img, &pl->map_tpl};
  for (int sl = 0; sl < pl->n_slabs; ++sl) {
    const int r0 = sl * pl->slab_rows;
    const int r1 = (r0 + pl->slab_rows < pl->HP) ? r0 + pl->slab_rows : pl->HP;
    a.q_begin = ct ? (r0 / v->CH) * nCWl : 0;
    a.q_end = ct ? (r1 / v->CH) * nCWl : a.nCH * a.nCW;
    a.c_row0 = r0;
    a.first = sl == 0;
    a.last = sl == pl->n_slabs - 1;
    const size_t cbytes = (size_t)(pl->n_tmpl > 1 ? (int64_t)pl->n_tmpl * pl->HP : (r1 - r0)) * pl->WP * 4;
    if (ct && pl->jit_ctpl) {  // the plan's own constant slot (JIT library): stream order suffices
      NCC_CUDA(cudaMemcpyAsync(pl->jit_ctpl, pl->tplC + (size_t)r0 * pl->WP, cbytes, cudaMemcpyDeviceToDevice, s));
      NCC_CUDA(cudaLaunchKernel(v->k[t][ct], grid, dim3(v->nt), args, (size_t)v->smem[t][ct], s));
    } else if (ct) {  // template rows [r0, r1) into the constant bank (stream-ordered after the prep)
      if (pl->capturing) {  // graph: the slot's ordering events wrap the graph launch (run_graph)
        NCC_CUDA(cudaMemcpyToSymbolAsync(c_tpl, pl->tplC + (size_t)r0 * pl->WP, cbytes, 0, cudaMemcpyDeviceToDevice, s));
        NCC_CUDA(cudaLaunchKernel(v->k[t][ct], grid, dim3(v->nt), args, (size_t)v->smem[t][ct], s));
      } else {
        ConstSlot& cs = g_const_slot[pl->device & 63];
        std::lock_guard<std::mutex> lk(cs.mu);
        if (!cs.done) NCC_CUDA(cudaEventCreateWithFlags(&cs.done, cudaEventDisableTiming));
        else NCC_CUDA(cudaStreamWaitEvent(s, cs.done, 0));
        NCC_CUDA(cudaMemcpyToSymbolAsync(c_tpl, pl->tplC + (size_t)r0 * pl->WP, cbytes, 0, cudaMemcpyDeviceToDevice, s));
        NCC_CUDA(cudaLaunchKernel(v->k[t][ct], grid, dim3(v->nt), args, (size_t)v->smem[t][ct], s));
        NCC_CUDA(cudaEventRecord(cs.done, s));
      }
    } else {
      NCC_CUDA(cudaLaunchKernel(v->k[t][ct], grid, dim3(v->nt), args, (size_t)v->smem[t][ct], s));
    }
  }
  mark(pl, s, 3);
  tm_finalize<<<ceil_div((int64_t)batch * pl->n_tmpl, 128), 128, 0, s>>>(
      pl->keys, pl->tst, pl->V, reinterpret_cast<PeakOut*>(d_peaks), batch, p.score == NCC_SCORE_SSD, pl->n_tmpl);
  mark(pl, s, 4);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return cuda_fail(e, "ncc_match launch");
  return NCC_OK;
}

// `npairs` pairs (<= the plan's batch) from A / B; vectors (and scores) of pair k at index k.
ncc_status run_piv(ncc_plan pl, const float* A, const float* B, float* d_scores, piv_vector* d_vec, cudaStream_t s,
                   int npairs = -1) {
  const ncc_problem& p = pl->p;
  const PivVariant* v = pl->pivv;
  const int batch = npairs < 0 ? p.batch : npairs;
  const int nsub = ceil_div(batch, pl->sub_batch);
  if (p.flags & NCC_F_TIMING) {
    ncc_status st = ensure_events(pl, 3 * nsub + 1);
    if (st) return st;
  }
  pl->timing_kind = 2;
  pl->piv_nsub = nsub;
  const int64_t fs = (int64_t)p.image_h * p.image_pitch;
  PivArgs a;
  a.A = A;
  a.B = B;
  a.pitch = p.image_pitch;
  a.frame_stride = fs;
  a.H = p.image_h;
  a.W = p.image_w;
  a.h = p.tmpl_h;
  a.w = p.tmpl_w;
  a.my = p.search_y;
  a.mx = p.search_x;
  a.sy = p.step_y;
  a.sx = p.step_x;
  a.Ky = pl->Ky;
  a.Kx = pl->Kx;
  a.S1 = pl->S1;
  a.S2 = pl->S2;
  a.map_pitch = pl->map_w;
  a.map_frame_stride = pl->s_frame_stride;
  a.vec = reinterpret_cast<VecOut*>(d_vec);
  a.scores = d_scores;
  a.subpix = p.subpix;
  a.BP = pl->piv_bp;
  a.ssd = p.score == NCC_SCORE_SSD;
  a.rsv = pl->tc_rsv;  // (only the warp-specialised kernels read them)
  a.mean = pl->tc_mean;
  // TMA maps over all frames of the call (3D: cols, rows, pair); plain loads otherwise
  CUtensorMap mB;
  memset(&mB, 0, sizeof(mB));
  // a TMA box must start on a 16-byte boundary of the row: window columns kx * step_x
  bool use_tma = v->k_tma != nullptr && p.image_pitch % 4 == 0 && p.step_x % 4 == 0 &&
                 reinterpret_cast<uintptr_t>(B) % 16 == 0;
  if (use_tma) {
    const uint64_t dims[3] = {(uint64_t)p.image_w, (uint64_t)p.image_h, (uint64_t)batch};
    const uint64_t strides[2] = {(uint64_t)p.image_pitch * 4, (uint64_t)fs * 4};
    const uint32_t boxB[3] = {(uint32_t)pl->piv_bp, (uint32_t)(p.tmpl_h + 2 * p.search_y), 1u};
    use_tma = boxB[1] <= 256 && boxB[0] <= 256 && encode_f32(&mB, B, 3, dims, strides, boxB);
  }
  CUtensorMap mW;  // the WS kernel's own box width
  memset(&mW, 0, sizeof(mW));
  if (use_tma && pl->ws_smem) {
    const uint64_t dims[3] = {(uint64_t)p.image_w, (uint64_t)p.image_h, (uint64_t)batch};
    const uint64_t strides[2] = {(uint64_t)p.image_pitch * 4, (uint64_t)fs * 4};
    const uint32_t boxB[3] = {(uint32_t)pl->ws_bp, (uint32_t)(p.tmpl_h + 2 * p.search_y), 1u};
    if (!(boxB[0] <= 256 && encode_f32(&mW, B, 3, dims, strides, boxB))) return NCC_ERR_CUDA;
  }
  CUtensorMap mT;  // tensor-core kernel: search-region rows, box (2 m_x + w, 1, 1)
  memset(&mT, 0, sizeof(mT));
  if (pl->ptc) {
    if (reinterpret_cast<uintptr_t>(B) % 16 != 0) return NCC_ERR_INVALID_ARGUMENT;  // (torch allocations are 256-B aligned)
    const uint64_t dims[3] = {(uint64_t)p.image_w, (uint64_t)p.image_h, (uint64_t)batch};
    const uint64_t strides[2] = {(uint64_t)p.image_pitch * 4, (uint64_t)fs * 4};
    const uint32_t box[3] = {(uint32_t)(2 * p.search_x + p.tmpl_w), 1u, 1u};
    if (!encode_f32(&mT, B, 3, dims, strides, box)) return NCC_ERR_CUDA;
  }
  const int groups = ceil_div((int64_t)pl->Ky * pl->Kx, v->WPB);
  mark(pl, s, 0);
  for (int sb = 0; sb < nsub; ++sb) {
    const int p0 = sb * pl->sub_batch;
    const int np = (p0 + pl->sub_batch <= batch) ? pl->sub_batch : batch - p0;
    if (pl->sad) {  // SAD: no window sums; frames of the sub-batch addressed from pair p0
      PivArgs as = a;
      as.A = A + p0 * fs;
      as.B = B + p0 * fs;
      as.pair0 = p0;
      mark(pl, s, 3 * sb + 1);
      piv_sad_kernel<<<dim3(pl->Ky * pl->Kx, np), 256, pl->sad_smem, s>>>(as);
      mark(pl, s, 3 * sb + 2);
      mark(pl, s, 3 * sb + 3);
      continue;
    }
    launch_box(pl, B + p0 * fs, np, 0, pl->map_h, s, false, pl->ptc && p.score == NCC_SCORE_NCC);  // the tensor-core PIV path reads only the fp32 factors
    mark(pl, s, 3 * sb + 1);
    a.pair0 = p0;
    dim3 grid(groups, 1, np);
    if (pl->ptc) {
      PivTcArgs t;
      t.A = A;
      t.pitch = p.image_pitch;
      t.frame_stride = fs;
      t.h = p.tmpl_h;
      t.w = p.tmpl_w;
      t.my = p.search_y;
      t.mx = p.search_x;
      t.sy = p.step_y;
      t.sx = p.step_x;
      t.Ky = pl->Ky;
      t.Kx = pl->Kx;
      t.pair0 = p0;
      t.Dx = 2 * p.search_x;
      t.R = pl->ptc_R;
      // column strips split into segments so that the launch has ~4 units per SM
      int nseg = (int)std::min<int64_t>(pl->Ky, std::max<int64_t>(1, ceil_div((int64_t)4 * pl->nsm, (int64_t)np * pl->Kx)));
      if (const char* e = getenv("NCC_PIV_TC_SEGW")) nseg = ceil_div(pl->Ky, std::max(1, atoi(e)));
      t.segw = ceil_div(pl->Ky, nseg);
      t.nseg = ceil_div(pl->Ky, t.segw);
      t.nunits = np * pl->Kx * t.nseg;
      t.rsv = pl->tc_rsv;
      t.mean = pl->tc_mean;
      t.map_pitch = pl->map_w;
      t.map_frame_stride = pl->s_frame_stride;
      t.border = pl->ptc_border;
      t.vec = reinterpret_cast<VecOut*>(d_vec);
      t.scores = d_scores;
      t.subpix = p.subpix;
      t.prof = pl->ptc_prof;
      t.nab = std::min(ptc::kNABMax, (512 - ptc::kNSlot * ptc::slot_cols(p.search_y, t.R)) / ptc::chunk_cols(p.tmpl_w));
      if (const char* e = getenv("NCC_PIV_TC_NAB")) t.nab = std::max(ptc::kNAB, std::min(t.nab, atoi(e)));
      t.exp = 0;
      if (const char* e = getenv("NCC_PIV_TC_EXP")) t.exp = atoi(e);
      if (pl->ptc_border_rb == 64)
        piv_tc_border_rb<64><<<dim3(pl->Ky * pl->Kx, np), 256 * (p.tmpl_w / 32), pl->ptc_border_smem, s>>>(t, B);
      else if (pl->ptc_border_rb == 32)
        piv_tc_border_rb<32><<<dim3(pl->Ky * pl->Kx, np), 256 * (p.tmpl_w / 32), pl->ptc_border_smem, s>>>(t, B);
      else
        piv_tc_border_kernel<<<dim3(pl->Ky * pl->Kx, np), 256, pl->ptc_border_smem, s>>>(t, B);
      void* targs[2] = {&t, &mT};
      const int g = std::min(t.nunits, pl->nsm);
      NCC_CUDA(cudaLaunchKernel((const void*)piv_tc_kernel, dim3(g), dim3(ptc::kThreads), targs, (size_t)pl->ptc_smem, s));
    } else if (use_tma && pl->ws_smem) {
      int total = (int)((int64_t)np * pl->Ky * pl->Kx);
      void* wargs[3] = {&a, &mW, &total};
      const int ngroups = ceil_div(total, v->ws_wps);
      const int g = ngroups < pl->ws_grid ? ngroups : pl->ws_grid;
      NCC_CUDA(cudaLaunchKernel(v->k_ws, dim3(g), dim3((v->ws_ncw + v->ws_npw) * 32), wargs, (size_t)pl->ws_smem, s));
    } else {
      void* args[2] = {&a, &mB};
      NCC_CUDA(cudaLaunchKernel(use_tma ? v->k_tma : v->k_ldg, grid, dim3(v->NT), args, (size_t)pl->piv_smem, s));
    }
    mark(pl, s, 3 * sb + 2);
    mark(pl, s, 3 * sb + 3);
  }
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return cuda_fail(e, "piv_correlate launch");
  return NCC_OK;
}

// Execute calls as CUDA graphs: the first call with a given set of pointer arguments captures
// the launch sequence (side-stream fork / join included) on the plan's capture stream and
// instantiates it; later calls replay it with one cudaGraphLaunch (no per-kernel launch cost,
// shorter gaps between dependent kernels).  Plans whose kernels read the device-wide constant
// template slot order the whole graph against other plans with the slot's event.
// NCC_NO_GRAPH=1 launches kernel by kernel.
bool is_pinned(const void* p) {  // page-locked (or device-accessible) host memory
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return a.type == cudaMemoryTypeHost || a.type == cudaMemoryTypeManaged;
}

bool graphs_disabled() {
  static const bool v = getenv("NCC_NO_GRAPH") != nullptr;
  return v;
}

template <class Body>
ncc_status run_graph(ncc_plan pl, const uintptr_t (&key)[8], cudaStream_t s, Body&& body) {
  if (graphs_disabled()) return body(s);
  int hit = -1;
  for (int k = 0; k < pl->n_graphs; ++k)
    if (memcmp(pl->graphs[k].key, key, sizeof(key)) == 0) hit = k;
  if (hit < 0) {
    if (!pl->cap) NCC_CUDA(cudaStreamCreateWithFlags(&pl->cap, cudaStreamNonBlocking));
    NCC_CUDA(cudaStreamBeginCapture(pl->cap, cudaStreamCaptureModeThreadLocal));
    pl->capturing = 1;
    const ncc_status st = body(pl->cap);
    pl->capturing = 0;
    cudaGraph_t g = nullptr;
    const cudaError_t e = cudaStreamEndCapture(pl->cap, &g);
    if (st != NCC_OK) {
      if (g) cudaGraphDestroy(g);
      cudaGetLastError();
      return st;
    }
    if (e != cudaSuccess) return cuda_fail(e, "graph capture");
    cudaGraphExec_t ex = nullptr;
    const bool fresh_slot = pl->n_graphs < 4;
    if (fresh_slot) {
      hit = pl->n_graphs++;
      pl->graphs[hit].exec = nullptr;
    } else {
      // evict round robin.  Callers rotating more than 4 buffer sets would otherwise pay a full
      // instantiation per call: the evicted executable is updated in place with the new graph
      // (same topology, new pointer arguments) when CUDA allows it; else re-instantiated.  (A
      // replay still in flight keeps the parameters it was launched with.)
      hit = pl->next_graph;
      pl->next_graph = (pl->next_graph + 1) % 4;
      cudaGraphExecUpdateResultInfo ui;
      if (cudaGraphExecUpdate(pl->graphs[hit].exec, g, &ui) == cudaSuccess) {
        ex = pl->graphs[hit].exec;
      } else {
        cudaGetLastError();
        cudaGraphExecDestroy(pl->graphs[hit].exec);
      }
      pl->graphs[hit].exec = nullptr;
    }
    if (!ex) {
      const cudaError_t ei = cudaGraphInstantiate(&ex, g, 0);
      if (ei != cudaSuccess) {
        cudaGraphDestroy(g);
        if (fresh_slot) --pl->n_graphs;                                   // slot unused again
        else memset(pl->graphs[hit].key, 0xFF, sizeof(pl->graphs[hit].key));  // never matches; exec null
        return cuda_fail(ei, "graph instantiate");
      }
    }
    cudaGraphDestroy(g);
    pl->graphs[hit].exec = ex;
    memcpy(pl->graphs[hit].key, key, sizeof(key));
    pl->graphs[hit].timing_kind = pl->timing_kind;
    pl->graphs[hit].piv_nsub = pl->piv_nsub;
  } else {
    pl->timing_kind = pl->graphs[hit].timing_kind;  // the replayed sequence's, not the last capture's
    pl->piv_nsub = pl->graphs[hit].piv_nsub;
  }
  const bool shared_const = pl->p.mode == NCC_MODE_MATCH && !pl->tc && !pl->tiny_fn && pl->use_ct && !pl->jit_ctpl;
  if (shared_const) {
    ConstSlot& cs = g_const_slot[pl->device & 63];
    std::lock_guard<std::mutex> lk(cs.mu);
    if (!cs.done) NCC_CUDA(cudaEventCreateWithFlags(&cs.done, cudaEventDisableTiming));
    else NCC_CUDA(cudaStreamWaitEvent(s, cs.done, 0));
    NCC_CUDA(cudaGraphLaunch(pl->graphs[hit].exec, s));
    NCC_CUDA(cudaEventRecord(cs.done, s));
  } else {
    NCC_CUDA(cudaGraphLaunch(pl->graphs[hit].exec, s));
  }
  return NCC_OK;
}

// The host paths' copy stream and slot events (lazy).
ncc_status ensure_copy_stream(ncc_plan pl) {
  if (pl->copy) return NCC_OK;
  NCC_CUDA(cudaStreamCreateWithFlags(&pl->copy, cudaStreamNonBlocking));
  for (int k = 0; k < 2; ++k) {
    NCC_CUDA(cudaEventCreateWithFlags(&pl->ev_copied[k], cudaEventDisableTiming));
    NCC_CUDA(cudaEventCreateWithFlags(&pl->ev_free[k], cudaEventDisableTiming));
  }
  NCC_CUDA(cudaEventCreateWithFlags(&pl->ev_start, cudaEventDisableTiming));
  return NCC_OK;
}

ncc_status stage(void** buf, size_t* have, size_t need) {
  if (*have >= need) return NCC_OK;
  cudaFree(*buf);
  *buf = nullptr;
  *have = 0;
  cudaError_t e = cudaMalloc(buf, need);
  if (e != cudaSuccess) {
    *buf = nullptr;
    return cuda_fail(e, "cudaMalloc(staging)");
  }
  *have = need;
  return NCC_OK;
}

}  // namespace

// ================================================================== extern "C"
extern "C" {

const char* ncc_status_string(ncc_status s) {
  switch (s) {
    case NCC_OK: return "NCC_OK";
    case NCC_ERR_INVALID_ARGUMENT: return "NCC_ERR_INVALID_ARGUMENT";
    case NCC_ERR_UNSUPPORTED: return "NCC_ERR_UNSUPPORTED";
    case NCC_ERR_OUT_OF_MEMORY: return "NCC_ERR_OUT_OF_MEMORY";
    case NCC_ERR_CUDA: return "NCC_ERR_CUDA";
    case NCC_ERR_COMPILE: return "NCC_ERR_COMPILE";
    case NCC_ERR_WRONG_MODE: return "NCC_ERR_WRONG_MODE";
  }
  return "NCC_ERR_UNKNOWN";
}

const char* ncc_last_cuda_error(void) { return g_last_cuda_error.c_str(); }

int32_t ncc_build_arch(void) { return 100; }

ncc_status ncc_specialize(const ncc_problem* p, char* variant_name, size_t name_size, int32_t* compiled_now) {
  if (!p) return NCC_ERR_INVALID_ARGUMENT;
  ncc_status st = validate(*p);
  if (st) return st;
  if (compiled_now) *compiled_now = 0;
  const int h = p->tmpl_h, w = p->tmpl_w, my = p->search_y, mx = p->search_x;
  std::string name;
  std::vector<std::string> names;
  if (p->mode == NCC_MODE_MATCH) {
    for (const TmVariant& c : kTmVariants)
      if (!(p->flags & NCC_F_GENERIC_KERNEL) && c.TH == h && c.TW == w) {
        name = c.name;
        break;
      }
    if (name.empty() && jit_allowed(p->flags)) {
      const TmJitChoice jc = tm_jit_choice(h, w);
      names = {tm_name(jc.RV, jc.LX, jc.WX, jc.WY, jc.CH, jc.CW, h, w, false, jc.ct),
               tm_name(jc.RV, jc.LX, jc.WX, jc.WY, jc.CH, jc.CW, h, w, true, jc.ct), "&nccb::c_tpl"};
      char b[96];
      snprintf(b, sizeof(b), "tm_jit_%dx%d_rv%d_lx%d_%dx%d_c%dx%d", h, w, jc.RV, jc.LX, jc.WY, jc.WX, jc.CH, jc.CW);
      name = b;
    }
    if (name.empty()) name = kTmVariants[0].name;
  } else {
    for (const PivVariant& c : kPivVariants)
      if (!(p->flags & NCC_F_GENERIC_KERNEL) && c.TH == h && c.TW == w && c.MY == my && c.MX == mx) name = c.name;
    if (name.empty() && jit_allowed(p->flags)) {
      const PivJitChoice jc = piv_jit_choice(h, w, my, mx);
      if (jc.ok) {
        names = {piv_name(h, w, my, mx, jc.RV, jc.CW, jc.NT, jc.WPB, jc.MINB, true, true, 1),
                 piv_name(h, w, my, mx, jc.RV, jc.CW, jc.NT, jc.WPB, jc.MINB, false, true, 1)};
        char b[96];
        snprintf(b, sizeof(b), "piv_jit_%dx%d_m%dx%d_rv%d_cw%d_nt%d_w%d", h, w, my, mx, jc.RV, jc.CW, jc.NT, jc.WPB);
        name = b;
      }
    }
    if (name.empty()) name = kPivVariants[0].name;
  }
  if (!names.empty()) {
    JitResult jr;
    std::string err;
    st = jit_build(names, &jr, &err);
    if (st) {
      g_last_cuda_error = err;
      return st;
    }
    if (compiled_now) *compiled_now = jr.cached ? 0 : 1;
  }
  if (variant_name && name_size) snprintf(variant_name, name_size, "%s", name.c_str());
  return NCC_OK;
}

ncc_status ncc_plan_create(const ncc_problem* p, int device, ncc_plan* out) {
  if (!out) return NCC_ERR_INVALID_ARGUMENT;
  *out = nullptr;
  if (!p) return NCC_ERR_INVALID_ARGUMENT;
  ncc_status st = validate(*p);
  if (st) return st;
  int ndev = 0;
  cudaError_t e = cudaGetDeviceCount(&ndev);
  if (e != cudaSuccess) return cuda_fail(e, "cudaGetDeviceCount");
  if (device < 0 || device >= ndev) return NCC_ERR_INVALID_ARGUMENT;
  DeviceGuard g(device);
  ncc_plan pl = new (std::nothrow) ncc_plan_s();
  if (!pl) return NCC_ERR_OUT_OF_MEMORY;
  pl->p = *p;
  pl->device = device;
  memset(&pl->info, 0, sizeof(pl->info));
  pl->info.mode = p->mode;
  pl->info.batch = p->batch;
  st = p->mode == NCC_MODE_MATCH ? create_tm(pl) : create_piv(pl);
  if (st) {
    free_plan(pl);
    return st;
  }
  *out = pl;
  return NCC_OK;
}

ncc_status ncc_plan_destroy(ncc_plan pl) {
  if (!pl) return NCC_OK;
  DeviceGuard g(pl->device);
  cudaDeviceSynchronize();
  free_plan(pl);
  return NCC_OK;
}

ncc_status ncc_plan_query(ncc_plan pl, void* info, size_t info_size) {
  if (!pl || !info) return NCC_ERR_INVALID_ARGUMENT;
  memcpy(info, &pl->info, info_size < sizeof(ncc_plan_info) ? info_size : sizeof(ncc_plan_info));
  return NCC_OK;
}

ncc_status ncc_plan_timing(ncc_plan pl, ncc_timing* out) {
  if (!pl || !out) return NCC_ERR_INVALID_ARGUMENT;
  memset(out, 0, sizeof(*out));
  if (!(pl->p.flags & NCC_F_TIMING) || pl->timing_kind == 0) return NCC_OK;
  DeviceGuard g(pl->device);
  float ms = 0.f;
  if (pl->timing_kind == 1) {
    NCC_CUDA(cudaEventSynchronize(pl->ev[4]));
    cudaEventElapsedTime(&ms, pl->ev[0], pl->ev[1]); out->prep_ms = ms;
    cudaEventElapsedTime(&ms, pl->ev[0], pl->ev[2]); out->stats_ms = ms;  // prep || window sums
    cudaEventElapsedTime(&ms, pl->ev[2], pl->ev[3]); out->numerator_ms = ms;
    cudaEventElapsedTime(&ms, pl->ev[3], pl->ev[4]); out->finalize_ms = ms;
    cudaEventElapsedTime(&ms, pl->ev[0], pl->ev[4]); out->total_ms = ms;
    out->numerator_launches = 1;
  } else {
    const int nsub = pl->piv_nsub;
    NCC_CUDA(cudaEventSynchronize(pl->ev[3 * nsub]));
    cudaEvent_t prev = pl->ev[0];
    for (int sb = 0; sb < nsub; ++sb) {
      cudaEventElapsedTime(&ms, prev, pl->ev[3 * sb + 1]); out->stats_ms += ms;
      cudaEventElapsedTime(&ms, pl->ev[3 * sb + 1], pl->ev[3 * sb + 2]); out->numerator_ms += ms;
      prev = pl->ev[3 * sb + 3];
    }
    cudaEventElapsedTime(&ms, pl->ev[0], pl->ev[3 * nsub]); out->total_ms = ms;
    out->numerator_launches = nsub;
  }
  return NCC_OK;
}

ncc_status ncc_match(ncc_plan pl, const float* d_images, const float* d_tmpl, int64_t tmpl_pitch, float* d_scores,
                     ncc_peak* d_peaks, void* stream) {
  if (!pl) return NCC_ERR_INVALID_ARGUMENT;
  if (pl->p.mode != NCC_MODE_MATCH || pl->roi_mode) return NCC_ERR_WRONG_MODE;
  if (!d_images || !d_tmpl || !d_peaks || tmpl_pitch < pl->p.tmpl_w) return NCC_ERR_INVALID_ARGUMENT;
  if ((pl->p.flags & NCC_F_WRITE_SURFACE) && !d_scores) return NCC_ERR_INVALID_ARGUMENT;
  DeviceGuard g(pl->device);
  const uintptr_t key[8] = {(uintptr_t)d_images, (uintptr_t)d_tmpl, (uintptr_t)tmpl_pitch, (uintptr_t)d_scores,
                            (uintptr_t)d_peaks, 0};
  return run_graph(pl, key, (cudaStream_t)stream, [&](cudaStream_t st) {
    return run_match(pl, d_images, d_tmpl, tmpl_pitch, d_scores, d_peaks, st);
  });
}

ncc_status ncc_match_rois(ncc_plan pl, const float* d_images, const float* d_tmpls, int64_t tmpl_pitch,
                          const int32_t* d_rois, float* d_scores, ncc_peak* d_peaks, void* stream) {
  if (!pl) return NCC_ERR_INVALID_ARGUMENT;
  if (pl->p.mode != NCC_MODE_MATCH || !pl->roi_mode) return NCC_ERR_WRONG_MODE;
  if (!d_images || !d_tmpls || !d_rois || !d_peaks || tmpl_pitch < pl->p.tmpl_w) return NCC_ERR_INVALID_ARGUMENT;
  if ((pl->p.flags & NCC_F_WRITE_SURFACE) && !d_scores) return NCC_ERR_INVALID_ARGUMENT;
  DeviceGuard g(pl->device);
  const uintptr_t key[8] = {(uintptr_t)d_images, (uintptr_t)d_tmpls, (uintptr_t)tmpl_pitch, (uintptr_t)d_scores,
                            (uintptr_t)d_peaks, (uintptr_t)d_rois};
  return run_graph(pl, key, (cudaStream_t)stream, [&](cudaStream_t st) {
    return run_match(pl, d_images, d_tmpls, tmpl_pitch, d_scores, d_peaks, st, d_rois);
  });
}

ncc_status piv_correlate_ex(ncc_plan pl, const float* d_a, const float* d_b, float* d_scores, piv_vector* d_vec,
                            void* stream) {
  if (!pl) return NCC_ERR_INVALID_ARGUMENT;
  if (pl->p.mode != NCC_MODE_PIV) return NCC_ERR_WRONG_MODE;
  if (!d_a || !d_b || !d_vec) return NCC_ERR_INVALID_ARGUMENT;
  DeviceGuard g(pl->device);
  const uintptr_t key[8] = {(uintptr_t)d_a, (uintptr_t)d_b, (uintptr_t)d_scores, (uintptr_t)d_vec,
                            (uintptr_t)pl->p.batch, 0};
  return run_graph(pl, key, (cudaStream_t)stream, [&](cudaStream_t st) {
    return run_piv(pl, d_a, d_b, d_scores, d_vec, st);
  });
}

ncc_status piv_correlate(ncc_plan pl, const float* d_a, const float* d_b, piv_vector* d_vec, void* stream) {
  return piv_correlate_ex(pl, d_a, d_b, nullptr, d_vec, stream);
}

ncc_status ncc_match_host(ncc_plan pl, const float* h_images, const float* h_tmpl, int64_t tmpl_pitch,
                          float* h_scores, ncc_peak* h_peaks, void* stream) {
  if (!pl) return NCC_ERR_INVALID_ARGUMENT;
  if (pl->p.mode != NCC_MODE_MATCH || pl->roi_mode) return NCC_ERR_WRONG_MODE;
  const ncc_problem& p = pl->p;
  if (!h_images || !h_tmpl || !h_peaks || tmpl_pitch < p.tmpl_w) return NCC_ERR_INVALID_ARGUMENT;
  DeviceGuard g(pl->device);
  cudaStream_t s = (cudaStream_t)stream;
  const size_t img_bytes = (size_t)p.batch * p.image_h * p.image_pitch * sizeof(float);
  const size_t t_bytes = (size_t)p.tmpl_h * p.tmpl_w * sizeof(float);
  const bool surf = (p.flags & NCC_F_WRITE_SURFACE) != 0;
  const size_t s_bytes = surf ? (size_t)p.batch * pl->Ub * pl->V * sizeof(float) : 0;
  ncc_status st;
  const bool pinned = is_pinned(h_images) && is_pinned(h_tmpl);
  // frames per streamed chunk: ~17 MB of frames (NCC_TM_CHUNK overrides; measured at cfg2, 8 frames
  // per call: chunks of 1 / 2 / 4 / 8 frames reach 57 / 60 / 70 / 65 % of the device-resident rate --
  // small chunks lose the batched numerator's efficiency, one chunk loses the overlap)
  const size_t frame_b = (size_t)p.image_h * p.image_pitch * sizeof(float);
  int chunk = (int)std::max<size_t>(1, ((size_t)17 << 20) / frame_b);
  if (const char* e = getenv("NCC_TM_CHUNK")) chunk = std::max(1, atoi(e));
  if (pinned && p.batch > chunk) {
    // Streaming (the paper's per-frame runtime operation, 5.1.3.4 P:91): chunks of
    // frames through two device slots -- the host->device copy of chunk c + 1 runs on the plan's
    // copy stream while chunk c is matched on `stream`; a slot is refilled only after its chunk's
    // peaks (and surfaces) were copied back.  The template is copied once per call.
    if ((st = ensure_copy_stream(pl))) return st;
    const size_t sframe_b = (size_t)pl->Ub * pl->V * sizeof(float);
    const size_t slot_b = (size_t)chunk * frame_b, sslot_b = surf ? (size_t)chunk * sframe_b : 0;
    const size_t pslot_b = (size_t)chunk * sizeof(ncc_peak);
    if ((st = stage((void**)&pl->st_a, &pl->st_a_bytes, 2 * slot_b))) return st;
    if ((st = stage((void**)&pl->st_t, &pl->st_t_bytes, t_bytes))) return st;
    if (surf && (st = stage((void**)&pl->st_s, &pl->st_s_bytes, 2 * sslot_b))) return st;
    if ((st = stage(&pl->st_out, &pl->st_out_bytes, 2 * pslot_b))) return st;
    NCC_CUDA(cudaMemcpy2DAsync(pl->st_t, p.tmpl_w * sizeof(float), h_tmpl, tmpl_pitch * sizeof(float),
                               p.tmpl_w * sizeof(float), p.tmpl_h, cudaMemcpyHostToDevice, s));
    NCC_CUDA(cudaEventRecord(pl->ev_start, s));  // earlier work on `stream` may still use the slots
    NCC_CUDA(cudaStreamWaitEvent(pl->copy, pl->ev_start, 0));
    const int nch = ceil_div(p.batch, chunk);
    for (int c = 0; c < nch; ++c) {
      const int k = c & 1, n = std::min(chunk, p.batch - c * chunk);
      float* sa = pl->st_a + (size_t)k * (slot_b / sizeof(float));
      float* ss = surf ? pl->st_s + (size_t)k * (sslot_b / sizeof(float)) : nullptr;
      ncc_peak* so = reinterpret_cast<ncc_peak*>(static_cast<char*>(pl->st_out) + (size_t)k * pslot_b);
      if (c >= 2) NCC_CUDA(cudaStreamWaitEvent(pl->copy, pl->ev_free[k], 0));
      NCC_CUDA(cudaMemcpyAsync(sa, reinterpret_cast<const char*>(h_images) + (size_t)c * slot_b, n * frame_b,
                               cudaMemcpyHostToDevice, pl->copy));
      NCC_CUDA(cudaEventRecord(pl->ev_copied[k], pl->copy));
      NCC_CUDA(cudaStreamWaitEvent(s, pl->ev_copied[k], 0));
      const uintptr_t key[8] = {(uintptr_t)sa, (uintptr_t)pl->st_t, (uintptr_t)p.tmpl_w, (uintptr_t)ss,
                                (uintptr_t)so, (uintptr_t)n, 0, 1};
      st = run_graph(pl, key, s, [&](cudaStream_t cs) {
        return run_match(pl, sa, pl->st_t, p.tmpl_w, ss, so, cs, nullptr, n);
      });
      if (st) return st;
      NCC_CUDA(cudaMemcpyAsync(h_peaks + (size_t)c * chunk, so, n * sizeof(ncc_peak), cudaMemcpyDeviceToHost, s));
      if (surf && h_scores)
        NCC_CUDA(cudaMemcpyAsync(reinterpret_cast<char*>(h_scores) + (size_t)c * chunk * sframe_b, ss,
                                 n * sframe_b, cudaMemcpyDeviceToHost, s));
      NCC_CUDA(cudaEventRecord(pl->ev_free[k], s));
    }
    return NCC_OK;
  }
  if ((st = stage((void**)&pl->st_a, &pl->st_a_bytes, img_bytes))) return st;
  if ((st = stage((void**)&pl->st_t, &pl->st_t_bytes, t_bytes))) return st;
  if (surf && (st = stage((void**)&pl->st_s, &pl->st_s_bytes, s_bytes))) return st;
  if ((st = stage(&pl->st_out, &pl->st_out_bytes, (size_t)p.batch * sizeof(ncc_peak)))) return st;
  if (pinned) {
    // pinned inputs: the copies are part of the (captured) launch sequence, the template's
    // ahead of its prep on the side stream (see run_match)
    const uintptr_t key[8] = {(uintptr_t)pl->st_a, (uintptr_t)pl->st_t, (uintptr_t)p.tmpl_w, (uintptr_t)pl->st_s,
                              (uintptr_t)pl->st_out, (uintptr_t)h_images, (uintptr_t)h_tmpl, (uintptr_t)tmpl_pitch};
    pl->h_img_in = h_images;
    pl->h_tmpl_in = h_tmpl;
    pl->h_tmpl_pitch = tmpl_pitch;
    st = run_graph(pl, key, s, [&](cudaStream_t cs) {
      return run_match(pl, pl->st_a, pl->st_t, p.tmpl_w, pl->st_s, (ncc_peak*)pl->st_out, cs);
    });
    pl->h_img_in = pl->h_tmpl_in = nullptr;
  } else {  // pageable inputs (staged copies, not capturable): copy, then the device-path graph
    NCC_CUDA(cudaMemcpyAsync(pl->st_a, h_images, img_bytes, cudaMemcpyHostToDevice, s));
    NCC_CUDA(cudaMemcpy2DAsync(pl->st_t, p.tmpl_w * sizeof(float), h_tmpl, tmpl_pitch * sizeof(float),
                               p.tmpl_w * sizeof(float), p.tmpl_h, cudaMemcpyHostToDevice, s));
    const uintptr_t key[8] = {(uintptr_t)pl->st_a, (uintptr_t)pl->st_t, (uintptr_t)p.tmpl_w, (uintptr_t)pl->st_s,
                              (uintptr_t)pl->st_out, 0};
    st = run_graph(pl, key, s, [&](cudaStream_t cs) {
      return run_match(pl, pl->st_a, pl->st_t, p.tmpl_w, pl->st_s, (ncc_peak*)pl->st_out, cs);
    });
  }
  if (st) return st;
  NCC_CUDA(cudaMemcpyAsync(h_peaks, pl->st_out, (size_t)p.batch * sizeof(ncc_peak), cudaMemcpyDeviceToHost, s));
  if (surf && h_scores) NCC_CUDA(cudaMemcpyAsync(h_scores, pl->st_s, s_bytes, cudaMemcpyDeviceToHost, s));
  return NCC_OK;
}

ncc_status piv_correlate_host(ncc_plan pl, const float* h_a, const float* h_b, piv_vector* h_vec, void* stream) {
  if (!pl) return NCC_ERR_INVALID_ARGUMENT;
  if (pl->p.mode != NCC_MODE_PIV) return NCC_ERR_WRONG_MODE;
  const ncc_problem& p = pl->p;
  if (!h_a || !h_b || !h_vec) return NCC_ERR_INVALID_ARGUMENT;
  DeviceGuard g(pl->device);
  cudaStream_t s = (cudaStream_t)stream;
  const size_t fb = (size_t)p.batch * p.image_h * p.image_pitch * sizeof(float);
  const size_t vb = (size_t)p.batch * pl->Ky * pl->Kx * sizeof(piv_vector);
  ncc_status st;
  const int chunk = pl->host_chunk;  // the copy / compute overlap granularity (<= the device sub-batch)
  if (p.batch <= chunk) {  // one chunk: copy in, run, copy out
    if ((st = stage((void**)&pl->st_a, &pl->st_a_bytes, fb))) return st;
    if ((st = stage((void**)&pl->st_b, &pl->st_b_bytes, fb))) return st;
    if ((st = stage(&pl->st_out, &pl->st_out_bytes, vb))) return st;
    NCC_CUDA(cudaMemcpyAsync(pl->st_a, h_a, fb, cudaMemcpyHostToDevice, s));
    NCC_CUDA(cudaMemcpyAsync(pl->st_b, h_b, fb, cudaMemcpyHostToDevice, s));
    const uintptr_t key[8] = {(uintptr_t)pl->st_a, (uintptr_t)pl->st_b, 0, (uintptr_t)pl->st_out,
                              (uintptr_t)p.batch, 0};
    st = run_graph(pl, key, s, [&](cudaStream_t cs) {
      return run_piv(pl, pl->st_a, pl->st_b, nullptr, (piv_vector*)pl->st_out, cs);
    });
    if (st) return st;
    NCC_CUDA(cudaMemcpyAsync(h_vec, pl->st_out, vb, cudaMemcpyDeviceToHost, s));
    return NCC_OK;
  }
  // Streaming: chunks of host_chunk pairs through two device slots.  The host->device copy of
  // chunk c + 1 runs on the plan's copy stream while chunk c is correlated on `stream`; a slot
  // is refilled only after the chunk that used it (and its vectors' copy-back) is done.
  if ((st = ensure_copy_stream(pl))) return st;
  const size_t pair_b = (size_t)p.image_h * p.image_pitch * sizeof(float);
  const size_t vpair_b = (size_t)pl->Ky * pl->Kx * sizeof(piv_vector);
  const size_t slot_b = (size_t)chunk * pair_b, vslot_b = (size_t)chunk * vpair_b;
  if ((st = stage((void**)&pl->st_a, &pl->st_a_bytes, 2 * slot_b))) return st;
  if ((st = stage((void**)&pl->st_b, &pl->st_b_bytes, 2 * slot_b))) return st;
  if ((st = stage(&pl->st_out, &pl->st_out_bytes, 2 * vslot_b))) return st;
  NCC_CUDA(cudaEventRecord(pl->ev_start, s));  // earlier work on `stream` may still use the slots
  NCC_CUDA(cudaStreamWaitEvent(pl->copy, pl->ev_start, 0));
  const int nch = ceil_div(p.batch, chunk);
  for (int c = 0; c < nch; ++c) {
    const int k = c & 1, n = std::min(chunk, p.batch - c * chunk);
    float* sa = pl->st_a + (size_t)k * (slot_b / sizeof(float));
    float* sb = pl->st_b + (size_t)k * (slot_b / sizeof(float));
    piv_vector* sv = reinterpret_cast<piv_vector*>(static_cast<char*>(pl->st_out) + (size_t)k * vslot_b);
    if (c >= 2) NCC_CUDA(cudaStreamWaitEvent(pl->copy, pl->ev_free[k], 0));
    NCC_CUDA(cudaMemcpyAsync(sa, h_a + (size_t)c * chunk * (pair_b / sizeof(float)), n * pair_b,
                             cudaMemcpyHostToDevice, pl->copy));
    NCC_CUDA(cudaMemcpyAsync(sb, h_b + (size_t)c * chunk * (pair_b / sizeof(float)), n * pair_b,
                             cudaMemcpyHostToDevice, pl->copy));
    NCC_CUDA(cudaEventRecord(pl->ev_copied[k], pl->copy));
    NCC_CUDA(cudaStreamWaitEvent(s, pl->ev_copied[k], 0));
    const uintptr_t key[8] = {(uintptr_t)sa, (uintptr_t)sb, 0, (uintptr_t)sv, (uintptr_t)n, 0};
    st = run_graph(pl, key, s, [&](cudaStream_t cs) { return run_piv(pl, sa, sb, nullptr, sv, cs, n); });
    if (st) return st;
    NCC_CUDA(cudaMemcpyAsync(reinterpret_cast<char*>(h_vec) + (size_t)c * chunk * vpair_b, sv, n * vpair_b,
                             cudaMemcpyDeviceToHost, s));
    NCC_CUDA(cudaEventRecord(pl->ev_free[k], s));
  }
  return NCC_OK;
}

}  // extern "C"
