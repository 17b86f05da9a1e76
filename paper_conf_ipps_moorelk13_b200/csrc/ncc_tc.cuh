// ncc_tc.cuh -- tensor-core (tcgen05, kind::f16, 3xBF16) numerator of the TM path.
//
// What it computes: the numerator stage of Fig 5.3, N[u][v] = sum_{i,j} A_C[i][j] *
// I[u+i][v+j], for a template block of up to HB x WC template elements; the normalisation
// (Figs 5.1/5.2) and the argmax stay in fp64 / fp32 exactly as in the CUDA-core path.
//
// Mapping onto the 5th-generation tensor cores (sm_100a):
//   * M = 128 output columns v of a tile (one TMEM lane each);
//   * K = template columns j, 16 per tcgen05.mma (bf16);
//   * N = a window of output rows u: for image row r the B operand row c is the template row
//     r - u(c), i.e. a window into the REVERSED, zero-padded template block held in shared
//     memory (K-major, no swizzle, 16-byte rows, so a window may start at any row: only the
//     descriptor start address moves); the accumulator D[v][u] lives in a ring of TMEM columns
//     indexed by u, and the MMA over image row r adds exactly the terms A_C[r-u][.] * I[r][v+.]
//     to every output row u of the window -- each output's sum accumulates in D in the same
//     row-by-row order, whatever band / segment the CTA works on (bitwise band-invariant).
//   * A operand = the Hankel matrix H_r[v][j] = I[r][v0+v+j] of image row r, written by the
//     producer warps straight into TMEM (tcgen05.st; lane v = row v), so the MMAs read only
//     the template window from shared memory.
//   * fp32-level accuracy from bf16 units: x = hi + lo + r (hi = bf16(x), lo = bf16(x - hi),
//     |r| <= 2^-17 |x|), A.B ~ A_hi.B_hi + A_hi.B_lo + A_lo.B_hi ("3xBF16"; each bf16 product exact
//     in the fp32 accumulator; per-product error ~2^-16 relative, random in sign, so ~2^-16 /
//     sqrt(h w) of the normalisation).  Round 1 used tf32 (3xTF32, K = 8): an M = 128 MMA costs
//     the same cycles for tf32 K = 8 and bf16 K = 16 (umma_probe rates), so 3xBF16 does the same
//     work in half the MMAs (cfg 5: 28.2 -> 21.5 ms; measured error at the planted peaks 1e-5 vs
//     2.25e-5 before: half as many accumulation steps).
// Rows are processed in groups of G: the window of group g is the HB + G output rows
// [G g - HB + 1, G g + G + 1); after the group the first G of them are complete, drained from
// TMEM (tcgen05.ld) to the partial-numerator buffer and their columns zeroed for reuse.
// Warp roles: warps 0-3 produce the Hankel operand (and drain the ring: lane quadrant w),
// warp 4 (one thread) issues the MMAs; TMEM A is double-buffered per (row, column chunk).
#pragma once
#include <cuda_bf16.h>
#include "ncc_kernels.cuh"

namespace nccb {
namespace tc {

__device__ __forceinline__ uint64_t sdesc(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
  uint64_t d = 0;
  d |= (uint64_t)((saddr >> 4) & 0x3FFFu);
  d |= (uint64_t)((lbo >> 4) & 0x3FFFu) << 16;
  d |= (uint64_t)((sbo >> 4) & 0x3FFFu) << 32;
  d |= (uint64_t)1 << 46;  // descriptor version (sm_100); base offset 0; SWIZZLE_NONE
  return d;
}
// kind::tf32 instruction descriptor: D f32, A/B tf32, both K-major, M = 128
__host__ __device__ constexpr uint32_t idesc_tf32(int N) {
  return (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);
}
__device__ __forceinline__ void mma_ts(uint32_t d, uint32_t a_tmem, uint64_t b, uint32_t idesc) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, 1, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::tf32 [%0], [%1], %2, %3, p;\n\t}" ::"r"(d),
      "r"(a_tmem), "l"(b), "r"(idesc)
      : "memory");
}
// kind::f16 instruction descriptor: D f32, A/B bf16, both K-major, M = 128
__host__ __device__ constexpr uint32_t idesc_bf16(int N) {
  return (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);
}
__device__ __forceinline__ void mma_bf16(uint32_t d, uint32_t a_tmem, uint64_t b, uint32_t idesc) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, 1, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n\t}" ::"r"(d),
      "r"(a_tmem), "l"(b), "r"(idesc)
      : "memory");
}
// Warp-wide forms for an issue loop run by all 32 lanes (warp-uniform operands stay on the uniform
// datapath): the instruction is issued once, by the lane elect.sync picks inside the asm -- no
// divergent C++ branch around it.
__device__ __forceinline__ void mma_bf16_warp(uint32_t d, uint32_t a_tmem, uint64_t b, uint32_t idesc) {
  asm volatile(
      "{\n\t.reg .pred E, A;\n\t"
      "elect.sync _|E, 0xffffffff;\n\t"
      "setp.ne.b32 A, 1, 0;\n\t"
      "@E tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, A;\n\t}" ::"r"(d),
      "r"(a_tmem), "l"(b), "r"(idesc)
      : "memory");
}
__device__ __forceinline__ void commit_warp(uint32_t bar) {
  asm volatile(
      "{\n\t.reg .pred E;\n\t"
      "elect.sync _|E, 0xffffffff;\n\t"
      "@E tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n\t}" ::"r"(bar)
      : "memory");
}
// x = hi + lo (+ r, |r| <= 2^-17 |x|): hi = bf16(x), lo = bf16(x - hi), packed (hi | lo << 16)
__device__ __forceinline__ uint32_t split_bf16(float x) {
  const __nv_bfloat16 h = __float2bfloat16_rn(x);
  const __nv_bfloat16 l = __float2bfloat16_rn(x - __bfloat162float(h));
  return (uint32_t)__bfloat16_as_ushort(h) | ((uint32_t)__bfloat16_as_ushort(l) << 16);
}
__device__ __forceinline__ void commit(uint64_t* bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(bar))
               : "memory");
}
__device__ __forceinline__ void fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void st_wait() { asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory"); }
__device__ __forceinline__ void st8(uint32_t addr, const uint32_t (&v)[8]) {
  asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"r"(addr), "r"(v[0]),
               "r"(v[1]), "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7])
               : "memory");
}
__device__ __forceinline__ void ld8(uint32_t addr, uint32_t (&v)[8]) {
  asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7])
               : "r"(addr)
               : "memory");
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}
// shared-window address forms (precomputed once: the generic -> shared conversion reads a
// special register, which the MMA issuer cannot afford between two MMAs)
__device__ __forceinline__ void commit_u32(uint32_t bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void mbar_wait_u32(uint32_t bar, uint32_t parity) {
  uint32_t done = 0;
  for (long long it = 0; it < (1ll << 30); ++it) {
    asm volatile(
        "{\n\t.reg .pred P;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 P, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, P;\n}"
        : "=r"(done)
        : "r"(bar), "r"(parity)
        : "memory");
    if (done) return;
  }
  __trap();
}
__device__ __forceinline__ bool mbar_try_u32(uint32_t bar, uint32_t parity) {
  uint32_t done;
  asm volatile(
      "{\n\t.reg .pred P;\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 P, [%1], %2;\n\t"
      "selp.u32 %0, 1, 0, P;\n}"
      : "=r"(done)
      : "r"(bar), "r"(parity)
      : "memory");
  return done != 0;
}
// mbarrier wait as ONE asm block: a non-blocking test_wait, and only on failure loop back (the
// success path falls through: no taken branch, no call between two MMAs of the issue loop; a
// satisfied try_wait measured ~350 cycles here).  Traps after ~2^30 failed polls (a hang guard, as
// mbar_wait_bounded).
__device__ __forceinline__ void mbar_wait_fall(uint32_t bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred P, Q;\n\t.reg .u32 n;\n\t"
      "mov.u32 n, 0;\n"
      "LAB_WAIT:\n\t"
      "mbarrier.test_wait.parity.shared::cta.b64 P, [%0], %1;\n\t"
      "@!P add.u32 n, n, 1;\n\t"
      "setp.gt.u32 Q, n, 1073741824;\n\t"
      "@Q trap;\n\t"
      "@!P bra LAB_WAIT;\n}"
      ::"r"(bar), "r"(parity)
      : "memory");
}
__device__ __forceinline__ bool elect_one() {
  uint32_t pred = 0;
  asm volatile("{\n\t.reg .pred P;\n\telect.sync _|P, 0xffffffff;\n\tselp.u32 %0, 1, 0, P;\n}" : "=r"(pred));
  return pred != 0;
}
__device__ __forceinline__ uint32_t to_tf32(float x) {
  uint32_t r;
  asm("cvt.rna.tf32.f32 %0, %1;" : "=r"(r) : "f"(x));
  return r;
}

constexpr int kHB = 128;   // template rows per block (B window rows N = kHB + kG)
constexpr int kG = 8;      // image rows per group (ring advance, drain granularity)
constexpr int kWB = 32;    // template columns per TMEM A chunk (4 MMAs of K = 8)
constexpr int kRing = 320; // TMEM accumulator columns (sliding window of output rows)
constexpr int kNBuf = 6;   // TMEM A stages (columns kRing + b*kWB .. ; 320 + 6*32 = 512): with bf16 operands a
                           // stage's MMAs take half as long, so more stages in flight hide the producers' latency
static_assert(kRing + kNBuf * kWB <= 512, "TMEM columns");  // A: kWB / 2 columns of bf16 pairs, hi and lo
constexpr int kNWin = kHB + kG;
// The window of group g starts at column (kG g) mod kRelocAt: when it would run past kRing the
// kHB live columns [kRelocAt, kRelocAt + kHB) are moved to [0, kHB) (relocation warps), so every
// MMA covers one contiguous run of columns (no ring-wrap split into two MMAs).
constexpr int kRelocAt = ((kRing - kNWin) / kG + 1) * kG;
static_assert(kRelocAt + kHB == kRing && kRelocAt >= kNWin, "relocation geometry");
// Row groups in flight between the MMA warp and the drain (epilogue) warps: the columns drained
// after group g are next written by the window of group g + kGRing (they enter it as its newest
// kG output rows: (kG g + kHB) mod kRelocAt == kG (g - kGRing)), so the MMA warp waits for the
// drain of group g - kGRing before group g; group-completion barriers form a ring of as many.
constexpr int kGRing = (kRelocAt - kHB) / kG;
static_assert(kGRing == 8 && ((kGRing * kG + kHB) % kRelocAt) == 0, "drain ring geometry");
constexpr int kLB = ((kHB + 2 * kG - 1 + 7) / 8) * 8;  // rows of the reversed template block
constexpr int kGroups = 2;  // producer groups of 4 warps; group g: stages q = g mod kGroups (2: with 16-load stages two
                           // groups keep ahead of the MMAs, and fewer warps share the issuer's SMSP)
// warp roles: producers 0 .. 4 kGroups - 1, relocation 4 kGroups .. + 3, TMA, then the MMA warp
// LAST: the SMSP arbiter issues highest-warp-id-first, and every cycle the MMA warp waits to issue
// is a cycle the tensor pipe idles (its queue is about one MMA deep).
constexpr int kRelocWarp0 = 4 * kGroups;   // 4 drain warps (TMEM lane quadrants): drain, zero, relocate
constexpr int kChainWarp0 = kRelocWarp0 + 4;  // 2 chain warps: the group's global work (64 columns each)
constexpr int kNChain = 2;
constexpr int kTmaWarp = kChainWarp0 + kNChain;
constexpr int kMmaWarp = kTmaWarp + 1;
constexpr int kThreads = kGroups * 128 + 128 + kNChain * 32 + 32 + 32;
constexpr int kBoxW = 128 + kWB;                         // image-row segment of one stage (TMA box)
constexpr int kNImg = 24;  // image-row ring (TMA issue distance: ~5 us of lookahead at cfg 2; 9 left the producers
                           // waiting ~760 cycles per stage for the data)
static_assert(kWB == 32 && kNBuf % 2 == 0 && kG % 2 == 0, "the WC = 32 issue loop: two K-steps of 16 per stage, stages in pairs of one phase");
static_assert(kNImg % kGroups == 0 && kNBuf % kGroups == 0, "a stage and the stage kNImg later belong to the same producer group");
// shared bytes of the template operand for a column super-block of WC columns (hi + lo)
__host__ __device__ constexpr uint32_t plane_bytes() { return kLB * 16; }
__host__ __device__ constexpr int b_bytes(int WC) { return 2 * (WC / 8) * kLB * 16; }  // bf16 hi + lo planes of 8
// dynamic shared memory per CTA: the operand, padded so that one CTA fits per SM (the CTA
// allocates all 512 TMEM columns)
__host__ __device__ constexpr int img_off(int WC) { return ((b_bytes(WC) + 127) / 128) * 128; }
// drained row groups staged for the chain warps: kGRing slots of kG rows x 128 columns (fp32)
// one ring slot: the stage's segment of the image operand as two planes of 8-byte elements (E, F),
// see tm_tc_split
constexpr int kSlotBytes = 2 * kBoxW * 8;
__host__ __device__ constexpr int stage_off(int WC) { return img_off(WC) + kNImg * kSlotBytes; }
__host__ __device__ constexpr int smem_need(int WC) { return stage_off(WC) + kGRing * kG * 128 * 4; }
__host__ __device__ constexpr int smem_bytes(int WC) { return smem_need(WC) > 120 * 1024 ? smem_need(WC) : 120 * 1024; }

}  // namespace tc

#ifdef NCC_TC_TRACE  // tools/microbench/tc_trace.cu: per-stage clock64 stamps of CTA 0
__device__ long long* g_tc_trace;
#ifdef NCC_TC_NOSTAMP
#define TC_STAMP(slot, q)
#else
#define TC_STAMP(slot, q) \
  if (blockIdx.x == 0 && blockIdx.y == 0 && (q) < 1024) g_tc_trace[(slot)*1024 + (q)] = clock64()
#endif
__device__ int g_tc_exp;  // timing experiments (trace builds only): bit0 no A stores, bit1 no wrap, bit2 one product
#define TC_EXP(bit) (g_tc_exp & (bit))
#else
#define TC_EXP(bit) 0
#define TC_STAMP(slot, q)
#endif

struct TcArgs {
  // the image operand of the band's rows (tm_tc_split: two planes of 8-byte pair elements per row),
  // read through the tensor map; H = absolute image rows (zero rows past it), u_begin = the band's first row
  int H, W;
  const float* tcB;     // [nblk][2 (hi, lo)][WC/4 planes][kLB rows][4]: reversed template blocks
  int WC;               // template columns per CTA (multiple of kWB, <= 128)
  int nbi, nbj;         // template blocks (row blocks of kHB, column super-blocks of WC)
  int V;                // output columns
  int u_begin, u_end;   // output rows of the band
  int useg, nseg;       // output rows per CTA segment, segments
  int vtiles;
  // Template blocks of one output tile accumulate in a fixed chain, block 0 -> nblk - 1 (no
  // partial planes, no summation kernel -- the paper's K2 global round trip, Figs 5.4-5.6, is
  // gone): block b > 0 adds its drained rows to the running numerator block b - 1 left in `acc`
  // (per-row-group, per-warp flags), the last block normalises them in the same drain.
  float* acc;              // [batch][u_end - u_begin][V] running numerator (one plane; chain mode)
  int planes;              // 1: planes mode -- the partial sums go to planes part + c part_blk_stride
  float* part;             //    (summed in plane order by tm_tc_finish); 0: the chain normalises in-kernel
  int clen;                // blocks per chain: planes mode 1 (plane c = block c), chain mode nblk (one chain);
                           // between: "chained planes" -- chains of clen blocks, plane c = chain c's sum
  int64_t acc_chain_stride;  // running-numerator plane of chain c: acc + c acc_chain_stride
  int64_t part_blk_stride;
  int64_t acc_frame_stride;
  unsigned int* flags;     // [batch][vtiles * nseg][ngrp_max][4]: blocks done with a row group
  int ngrp_max;
  unsigned long long* ticket;  // monotonically increasing CTA ticket (start order -> chain order)
  const double *S1, *S2;   // fp64 window sums [batch][u_end - u_begin][V] (box2d; SSD)
  const float *rsv, *mean; // NCC: fp32 rsqrt(n var) (0: flat window) and S1/n per offset (same layout)
  int64_t stat_frame_stride;
  const TemplateStats* tst;
  int h, w;
  float* scores;           // optional surface [batch][u_end - u_begin][V]
  int64_t score_frame_stride;
  unsigned long long* keys;  // per-frame packed argmax keys
  int ssd;
  int center;  // the image operand is centred on the template mean (tm_tc_split with ts)
  unsigned long long* prof;  // NCC_TC_EXP bit 32: per-CTA wait accounting [ticket][8] (globaltimer ns)
  const int32_t* rois;     // ROI mode (planes): [frame][template][2] offset-space origins; else nullptr
  int n_tmpl, roi_h, roi_w, U;
  int exp;  // timing experiments (NCC_TC_EXP; 0 in normal use): 1 no chain waits, 2 no drain work,
            // 16 prefetch only (no chain / normalisation work)
};

// Centring constant of the image operand: the template mean as an fp32 value (the same value in
// tm_tc_split and in the epilogue's correction).
__host__ __device__ __forceinline__ float tc_center(const TemplateStats* ts, double n) {
  return ts ? (float)(ts->sum / n) : 0.0f;
}
__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}
__device__ __forceinline__ unsigned int ld_acquire_u32(const unsigned int* p) {
  unsigned int v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_u32(unsigned int* p, unsigned int v) {
  asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

// grid = (nblk * vtiles * nseg, batch); block = tc::kThreads; dynamic smem = tc::b_bytes(WC).
__global__ void __launch_bounds__(tc::kThreads, 1) tm_tc_kernel(const TcArgs a,
                                                                  const __grid_constant__ CUtensorMap map_img) {
  using namespace tc;
  extern __shared__ __align__(1024) unsigned char smem_tc[];
  __shared__ __align__(8) uint64_t a_full[kNBuf], mma_done[kNBuf], img_full[kNImg], img_empty[kNImg], reloc_req,
      reloc_done, grp_done[kGRing], drained[kGRing], staged[kGRing], consumed[kGRing];
  __shared__ uint32_t tmem_base_s;
  __shared__ unsigned long long ticket_s;

  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int nblk = a.nbi * a.nbj;
  // The CTA's work comes from a ticket taken when it starts, template block fastest: the CTA of
  // block b of a tile always started after the one of block b - 1 (which it may wait for), so
  // the chain never waits on a CTA that is not resident or finished, whatever the hardware's
  // dispatch order.  The counter only grows: a launch of this plan always has the same grid.
  if (tid == 0) ticket_s = atomicAdd(a.ticket, 1ull) % ((unsigned long long)gridDim.x * gridDim.y);
  // a kernel launched after this one as its programmatic dependent (planes mode: the window sums,
  // which read only the frames) may start now, on the SMs this grid leaves free
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  __syncthreads();
  const int64_t tk = (int64_t)ticket_s;
  const int blk = (int)(tk % nblk);
  const int64_t rest = tk / nblk;
  const int tile = (int)(rest % ((int64_t)a.vtiles * a.nseg));  // = seg * vtiles + vt
  const int vt = tile % a.vtiles, seg = tile / a.vtiles;
  const int bi = blk / a.nbj, bj = blk % a.nbj;
  // sub-problem: a frame (plain band matching) or a (frame, template) pair with its ROI
  const int f = (int)(rest / ((int64_t)a.vtiles * a.nseg));  // sub-problem index
  int frm = f, tt = 0, ru0 = a.u_begin, uend = a.u_end, rv0 = 0, vend = a.V, opitch = a.V;
  int64_t osub = a.acc_frame_stride;
  if (a.rois) {  // ROI mode (planes): the ROI origin of (frame, template) from device memory
    frm = f / a.n_tmpl;
    tt = f % a.n_tmpl;
    ru0 = min(max(a.rois[2 * f], 0), a.U - 1);
    rv0 = min(max(a.rois[2 * f + 1], 0), a.V - 1);
    uend = min(ru0 + a.roi_h, a.U);
    vend = min(rv0 + a.roi_w, a.V);
    opitch = a.roi_w;
    osub = (int64_t)a.roi_h * a.roi_w;
  }
  // (a TMA box of 8-byte (hi, lo) elements must start 16-byte aligned: ROI tiles start at the even
  // column at or below the ROI origin, one more tile covers the shift, the extra column is masked)
  const int v0 = (rv0 & ~3) + vt * 128;
  const int ua = ru0 + seg * a.useg;
  const int nu = max(0, min(a.useg, uend - ua));  // output rows of this CTA
  const int i0 = bi * kHB, j0 = bj * a.WC;
  const int nch = a.WC / kWB;                // TMEM chunks per image row
  const int R = nu + kHB - 1;                // image rows touching the CTA's outputs
  const int ngrp = nu > 0 ? (R + kG - 1) / kG : 0;
  const int nrow = ngrp * kG;
  const int nstage = nrow * nch;             // (row, chunk) stages
  const uint32_t plane = kLB * 16;           // bytes per K plane of the template operand
  const int npl = a.WC / 8;  // bf16 K planes (8 columns of 16 bytes)

  // template operand (precomputed layout) -> shared memory
  {
    const float4* src = reinterpret_cast<const float4*>(a.tcB + ((int64_t)tt * nblk + blk) * (b_bytes(a.WC) / 4));
    float4* dst = reinterpret_cast<float4*>(smem_tc);
    const int n4 = b_bytes(a.WC) / 16;
    for (int k = tid; k < n4; k += kThreads) dst[k] = __ldg(src + k);
  }
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_u32(&tmem_base_s)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (tid == 0) {
    for (int b = 0; b < kNBuf; ++b) {
      mbar_init(&a_full[b], 128);
      mbar_init(&mma_done[b], 1);
    }
    for (int b = 0; b < kNImg; ++b) {
      mbar_init(&img_full[b], 1);
      mbar_init(&img_empty[b], 128);
    }
    mbar_init(&reloc_req, 1);
    mbar_init(&reloc_done, 128);
    for (int b = 0; b < kGRing; ++b) {
      mbar_init(&grp_done[b], 1);   // tcgen05.commit after a row group's last MMA
      mbar_init(&drained[b], 128);  // the group's accumulator columns read and zeroed
      mbar_init(&staged[b], 128);   // the group's values in the shared-memory slot (drain warps)
      mbar_init(&consumed[b], kNChain * 32);  // ... read by the chain warps: the slot is free
    }
    fence_mbar_init();
  }
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t tbase = tmem_base_s;
  const uint32_t a_col0 = kRing;  // A buffers: [kRing + b*2*kWB, +kWB) hi, [+kWB, +2kWB) lo

  // stage q = (image row rr, column chunk ch): row ua + i0 + rr, columns v0 + j0 + 32 ch + [0, kBoxW)
  auto stage_zero = [&](int q) {  // rows past the image / chunks past its width: zero operand
    if (nch == 1) return ua + i0 + q >= a.H || v0 + j0 >= a.W;
    return ua + i0 + q / nch >= a.H || v0 + j0 + (q % nch) * kWB >= a.W;
  };
  auto issue = [&](int q) {  // one thread: TMA of stage q into ring slot q % kNImg
    const int sl = q % kNImg;
    if (q >= kNImg) mbar_wait_bounded(&img_empty[sl], (uint32_t)(((q - kNImg) / kNImg) & 1));
    if (stage_zero(q)) {
      mbar_arrive(&img_full[sl]);
    } else {
      mbar_expect_tx(&img_full[sl], (uint32_t)kSlotBytes);
      tma_load_4d(smem_tc + img_off(a.WC) + sl * kSlotBytes, &map_img, v0 + j0 + (nch == 1 ? 0 : q % nch) * kWB, 0,
                  ua - a.u_begin + i0 + (nch == 1 ? q : q / nch), frm, &img_full[sl]);
    }
  };
  if (TC_EXP(32768) && warp != kMmaWarp) {
    // trace experiment: the MMA warp alone
  } else if (TC_EXP(65536) && warp < 4 * kGroups) {
    // trace experiment: no producers (TMA and relocation warps still run)
    if (warp == 0) {
      for (int q = 0; q < nstage; ++q) {  // keep the TMA ring moving
        const int sl = q % kNImg;
        mbar_wait_bounded(&img_full[sl], (uint32_t)((q / kNImg) & 1));
        if (lane == 0) for (int k = 0; k < 128; ++k) mbar_arrive(&img_empty[sl]);
        __syncwarp();
      }
    }
  } else if (warp < 4 * kGroups) {
    // ===================== producers (lane v = output column v0 + v).
    // Group grp (warps 4 grp .. 4 grp + 3, TMEM lane quadrants 0..3) handles the stages
    // q = grp mod kGroups (TMEM A buffer q mod kNBuf): the groups' latencies overlap.
    const int grp = warp >> 2, wq = warp & 3;
    const int gtid = tid & 127;  // thread index within the group
    const uint32_t lane_base = (uint32_t)(wq * 32) << 16;
    const int v = wq * 32 + lane;
    if (grp == 0) {  // zero the accumulator ring before the first MMA (ordered by group 0's a_full arrival)
      const uint32_t z[8] = {0u, 0u, 0u, 0u, 0u, 0u, 0u, 0u};
#pragma unroll 1
      for (int c = 0; c < kRing; c += 8) st8(tbase + lane_base + c, z);
      st_wait();
      fence_before();
    }
    const uint2* ring = reinterpret_cast<const uint2*>(smem_tc + img_off(a.WC));
    // Software-pipelined producer: the operand of the group's next stage is read from the ring
    // while the group waits for its TMEM buffer, so the critical path from "MMAs of the buffer's
    // previous stage done" to "a_full" is only the TMEM stores (the MMA warp has kNBuf - 1 stages
    // of slack).  (Finished row groups are drained by the epilogue warps.)
    uint32_t hi[kWB / 2], lo[kWB / 2];  // bf16 pairs (element 2p in the low half)
    auto load_split = [&](int q) {
      const int sl = q % kNImg;
      mbar_wait_bounded(&img_full[sl], (uint32_t)((q / kNImg) & 1));
      if (gtid == 0) TC_STAMP(5, q);
      // tm_tc_split stored, per image element k, E_k = (P_k, P_{k+2}) and F_k = (Q_k, Q_{k+2}) with
      // P_k = (bf16 hi_k | hi_{k+1} << 16), Q_k the same of lo: the lane's Hankel row is 8 loads of 8
      // bytes from each plane (elements v, v + 4, ..., v + 28), already in MMA operand order -- no
      // shifts, selects or permutes (the producers' instruction count sets the stage time: their
      // warps share the SMSPs with the MMA issuer).  A warp's load covers 32 consecutive 8-byte
      // elements: 2 wavefronts, no conflicts.
      const bool zero = stage_zero(q) || TC_EXP(64);
      const uint2* e = ring + sl * 2 * kBoxW + v;
#pragma unroll
      for (int m = 0; m < kWB / 4; ++m) {
        const uint2 th = zero ? make_uint2(0u, 0u) : e[4 * m];
        const uint2 tl = zero ? make_uint2(0u, 0u) : e[kBoxW + 4 * m];
        hi[2 * m] = th.x;
        hi[2 * m + 1] = th.y;
        lo[2 * m] = tl.x;
        lo[2 * m + 1] = tl.y;
      }
      mbar_arrive(&img_empty[sl]);
      if (gtid == 0) TC_STAMP(1, q);
    };
    if (grp < nstage) load_split(grp);
#pragma unroll 1
    for (int q = grp; q < nstage + kNBuf; q += kGroups) {
      const int b = q % kNBuf;
      const int qd = q - kNBuf;  // the buffer's previous stage
      if (qd >= 0) {
        if (!TC_EXP(256)) mbar_wait_bounded(&mma_done[b], (uint32_t)((qd / kNBuf) & 1));
        if (!TC_EXP(128)) fence_after();
        if (gtid == 0) TC_STAMP(0, qd);
      }
      if (q < nstage) {
        const uint32_t ab = tbase + lane_base + a_col0 + (uint32_t)(b * kWB);
        if (!TC_EXP(1)) {  // [kWB / 2 columns of hi pairs][kWB / 2 of lo pairs]
#pragma unroll
          for (int c = 0; c < kWB / 2; c += 8) {
            st8(ab + c, *reinterpret_cast<const uint32_t(*)[8]>(hi + c));
            st8(ab + kWB / 2 + c, *reinterpret_cast<const uint32_t(*)[8]>(lo + c));
          }
        }
        if (!TC_EXP(512)) st_wait();
        if (!TC_EXP(128)) fence_before();
        mbar_arrive(&a_full[b]);
        if (gtid == 0) TC_STAMP(2, q);
      }
      if (q + kGroups < nstage) load_split(q + kGroups);
    }
  } else if (warp == kTmaWarp) {
    // ===================== TMA producer: image-row segments, kNImg stages ahead
    if (lane == 0) {
      tma_prefetch_desc(&map_img);
#pragma unroll 1
      for (int q = 0; q < nstage; ++q) issue(q);
    }
    __syncwarp();
  } else if (warp >= kRelocWarp0 && warp < kRelocWarp0 + 4) {
    // ===================== drain warps (lane quadrant wq = warp % 4, lane = column v0 + 32 wq + lane):
    // for every finished row group read its kG accumulator columns from TMEM, zero them and
    // release them to the MMA warp (drained ring), then stage the values in shared memory for the
    // chain warps (staged / consumed ring); between groups, the rare relocation of the live
    // window.  No global memory traffic here, so nothing the MMA warp waits for depends on
    // another CTA.
    const int wq = warp & 3;
    const uint32_t lane_base = (uint32_t)(wq * 32) << 16;
    const uint32_t z[8] = {0u, 0u, 0u, 0u, 0u, 0u, 0u, 0u};
    float* stg = reinterpret_cast<float*>(smem_tc + stage_off(a.WC)) + wq * 32 + lane;
    int nrel = 0;
#pragma unroll 1
    for (int gd = 0; gd < ngrp; ++gd) {
      if (gd > 0 && (gd * kG) % kRelocAt == 0) {
        // the MMA warp requests the relocation before group gd (all earlier MMAs complete, all
        // earlier groups drained by these warps): move the live columns to the front
        mbar_wait_bounded(&reloc_req, (uint32_t)(nrel & 1));
        fence_after();
#pragma unroll 1
        for (int c = 0; c < kHB; c += 8) {
          uint32_t d[8];
          ld8(tbase + lane_base + kRelocAt + c, d);
          st8(tbase + lane_base + c, d);
          st8(tbase + lane_base + kRelocAt + c, z);
        }
        st_wait();
        fence_before();
        mbar_arrive(&reloc_done);
        ++nrel;
      }
      mbar_wait_bounded(&grp_done[gd % kGRing], (uint32_t)((gd / kGRing) & 1));
      fence_after();
      const uint32_t col = (uint32_t)((gd * kG) % kRelocAt);
      uint32_t d[8];
      ld8(tbase + lane_base + col, d);
      st8(tbase + lane_base + col, z);  // the columns are free again once read
      st_wait();
      fence_before();
      mbar_arrive(&drained[gd % kGRing]);
      const int slot = gd % kGRing;
      if (gd >= kGRing) mbar_wait_bounded(&consumed[slot], (uint32_t)(((gd - kGRing) / kGRing) & 1));
      float* sp = stg + slot * (kG * 128);
#pragma unroll
      for (int k = 0; k < kG; ++k) sp[k * 128] = __uint_as_float(d[k]);
      mbar_arrive(&staged[slot]);
    }
  } else if (warp >= kChainWarp0 && warp < kChainWarp0 + kNChain) {
    // ===================== chain warps: lane = columns v0 + 64 cw + 32 j + lane (j = 0, 1).
    // Row group gd holds output rows up = kG gd - kHB + 1 + k, k < kG.  Chain: block b > 0 adds
    // its values to the running numerator block b - 1 published for the group (per chain warp
    // flag); blocks b < nblk - 1 publish the new running value; the last block normalises (fp32
    // from the window kernels' fp64-derived factors), writes the surface and folds the argmax
    // keys.  Per output the order is ((p_0 + p_1) + p_2) + ... in block order: deterministic and
    // independent of bands and segments.
    const int cw = warp - kChainWarp0;
    const bool last_blk = blk == nblk - 1;
    // chain of this block (chained planes: the plane index too) and its position in the chain
    const int cid = blk / a.clen, nchains = (nblk + a.clen - 1) / a.clen;
    const bool chained = a.clen > 1, cfirst = blk % a.clen == 0, clast = blk % a.clen == a.clen - 1 || last_blk;
    auto flag_ptr = [&](int g) {
      return a.flags + (((int64_t)(f * a.vtiles * a.nseg + tile) * nchains + cid) * a.ngrp_max + g) * 4 + cw;
    };
    const float* stg = reinterpret_cast<const float*>(smem_tc + stage_off(a.WC)) + cw * 64 + lane;
    unsigned long long* prof = (a.exp & 32) && lane == 0 && cw == 0 ? a.prof + (int64_t)tk * 8 : nullptr;
    unsigned long long p_flag = 0, p_grp = 0, p_chain = 0;
    unsigned long long wbest = 0ull;  // last block: this lane's best key over its groups
    int pending = -1;                 // group whose running sums are stored but not yet flagged
    const double inv_n = 1.0 / ((double)a.h * (double)a.w);
    int vcol[2];
    bool colok[2];
    int64_t cb[2];  // offset of (the CTA's first output row, this column) in a frame's [Ub][V] planes
#pragma unroll
    for (int j = 0; j < 2; ++j) {
      vcol[j] = v0 + cw * 64 + 32 * j + lane;
      colok[j] = vcol[j] >= rv0 && vcol[j] < vend;
      cb[j] = (int64_t)(ua - ru0) * opitch + ((colok[j] ? vcol[j] : rv0) - rv0);
    }
    float* accb = chained ? a.acc + (int64_t)f * a.acc_frame_stride + (int64_t)cid * a.acc_chain_stride : nullptr;
    const int64_t sfo = (int64_t)f * a.stat_frame_stride;
#pragma unroll 1
    for (int gd = 0; gd < ngrp; ++gd) {
      const int up0 = gd * kG - kHB + 1;
      const bool has_rows = up0 + kG > 0 && up0 < nu && !TC_EXP(32) && !(a.exp & 2);
      const int slot = gd % kGRing;
      unsigned int* fl = flag_ptr(gd);
      unsigned long long pt = prof ? gtimer() : 0ull;
      int64_t rowoff[kG];
#pragma unroll
      for (int k = 0; k < kG; ++k) rowoff[k] = (int64_t)min(max(up0 + k, 0), nu - 1) * a.V;
      float prev[2][kG], fa[2][kG], fb[2][kG];
      if (has_rows && last_blk && !a.ssd && !a.planes) {  // normalisation factors: requested first
#pragma unroll
        for (int j = 0; j < 2; ++j)
#pragma unroll
          for (int k = 0; k < kG; ++k) {
            fa[j][k] = __ldcg(a.rsv + sfo + cb[j] + rowoff[k]);
            fb[j][k] = __ldcg(a.mean + sfo + cb[j] + rowoff[k]);
          }
      }
      // Software-pipelined chain: the running sums of group gd - 1 were stored at the end of the
      // previous iteration; their flag is published here, its fence overlapping the first poll of
      // this group's predecessor flag (two L2 round trips per group instead of three).
      auto publish_pending = [&]() {
        if (pending >= 0) {
          __threadfence();  // each lane's stores before the flag (the threadFenceReduction pattern)
          __syncwarp();
          if (lane == 0) st_release_u32(flag_ptr(pending), (unsigned)(blk + 1));
          pending = -1;
        }
      };
      if (has_rows && chained && !cfirst && !(a.exp & 1)) {  // every lane acquires the flag itself
        unsigned int fv = ld_acquire_u32(fl);
        publish_pending();
        for (long long it = 0; fv < (unsigned)blk; ++it) {
          if (it > (1ll << 28)) __trap();
          fv = ld_acquire_u32(fl);
        }
      } else {
        publish_pending();
      }
      if (prof) { const unsigned long long t = gtimer(); p_flag += t - pt; pt = t; }
      if (has_rows && chained && !cfirst) {
#pragma unroll
        for (int j = 0; j < 2; ++j)
#pragma unroll
          for (int k = 0; k < kG; ++k) prev[j][k] = __ldcg(accb + cb[j] + rowoff[k]);
      }
      mbar_wait_bounded(&staged[slot], (uint32_t)((gd / kGRing) & 1));
      if (prof) { const unsigned long long t = gtimer(); p_grp += t - pt; pt = t; }
      float x[2][kG];
#pragma unroll
      for (int j = 0; j < 2; ++j)
#pragma unroll
        for (int k = 0; k < kG; ++k) x[j][k] = stg[slot * (kG * 128) + k * 128 + 32 * j];
      mbar_arrive(&consumed[slot]);
      if (has_rows && a.planes && !chained) {  // planes mode: this block's partial sums to its own plane (no waiting)
        float* pb = a.part + (int64_t)blk * a.part_blk_stride + (int64_t)f * osub;
#pragma unroll
        for (int j = 0; j < 2; ++j)
#pragma unroll
          for (int k = 0; k < kG; ++k) {
            const int up = up0 + k;
            if (up >= 0 && up < nu && colok[j]) __stcg(pb + cb[j] + (int64_t)up * opitch, x[j][k]);
          }
      } else if (has_rows && !(a.exp & 16)) {
        if (!cfirst) {
#pragma unroll
          for (int j = 0; j < 2; ++j)
#pragma unroll
            for (int k = 0; k < kG; ++k) x[j][k] = prev[j][k] + x[j][k];
        }
        if (clast && a.planes) {  // chained planes: the chain's sum to plane cid (tm_tc_finish)
          float* pb = a.part + (int64_t)cid * a.part_blk_stride + (int64_t)f * osub;
#pragma unroll
          for (int j = 0; j < 2; ++j)
#pragma unroll
            for (int k = 0; k < kG; ++k) {
              const int up = up0 + k;
              if (up >= 0 && up < nu && colok[j]) __stcg(pb + cb[j] + (int64_t)up * opitch, x[j][k]);
            }
          if (lane == 0 && !cfirst) *fl = 0u;  // consumed: ready for the next call (stream-ordered)
        } else if (!clast) {
#pragma unroll
          for (int j = 0; j < 2; ++j)
#pragma unroll
            for (int k = 0; k < kG; ++k) {
              const int up = up0 + k;
              if (up >= 0 && up < nu && colok[j]) __stcg(accb + cb[j] + (int64_t)up * a.V, x[j][k]);
            }
          pending = gd;  // published at the start of the next iteration (or after the loop)
        } else {
          const TemplateStats ts = a.tst[0];
          // centred operand: sum A_C I = sum A_C (I - c) + c sum A_C
          const double dc = a.center ? (double)tc_center(&ts, (double)a.h * (double)a.w) * ts.csum : 0.0;
          const float csf = (float)ts.csum, dcf = (float)dc;
          const float rse = ts.flat ? 0.0f : (float)(1.0 / sqrt(ts.energy));
#pragma unroll
          for (int j = 0; j < 2; ++j) {
            const int vv = vcol[j];
#pragma unroll
            for (int k = 0; k < kG; ++k) {
              float sc;
              if (a.ssd) {
                const double num = (double)x[j][k] + dc;
                sc = (float)(ts.sumsq - 2.0 * (num + ts.sum * inv_n * __ldcg(a.S1 + sfo + cb[j] + rowoff[k])) + __ldcg(a.S2 + sfo + cb[j] + rowoff[k]));
              } else {  // |error| <= ~3e-7: three fp32 roundings of fp64-derived factors
                const float r = (a.exp & 64) ? x[j][k] : fmaf(-csf, fb[j][k], x[j][k] + dcf) * (fa[j][k] * rse);
                sc = r > 1.0f ? 1.0f : (r < -1.0f ? -1.0f : r);
              }
              const int up = up0 + k;
              if (up >= 0 && up < nu && colok[j]) {
                if (a.scores) a.scores[(int64_t)f * a.score_frame_stride + cb[j] + (int64_t)up * a.V] = sc;
                const unsigned long long key = make_key(a.ssd ? -sc : sc, (uint32_t)((int64_t)(ua + up) * a.V + vv));
                wbest = key > wbest ? key : wbest;
              }
            }
          }
          if (lane == 0 && !cfirst) *fl = 0u;  // consumed: ready for the next call (stream-ordered)
        }
      }
      if (prof) {
        const unsigned long long t = gtimer();
        p_chain += t - pt;
        if (tk < 4 && gd < 64) {  // per-group trace of the first tile's CTAs: [ticket][gd] chain done
          unsigned long long* tr = a.prof + (int64_t)gridDim.x * gridDim.y * 8;
          tr[tk * 64 + gd] = t;
        }
      }
    }
    if (pending >= 0) {  // the last group's running sums
      __threadfence();
      __syncwarp();
      if (lane == 0) st_release_u32(flag_ptr(pending), (unsigned)(blk + 1));
    }
    if (last_blk && !a.planes) {
      wbest = warp_max_key(wbest);
      if (lane == 0 && wbest) atomicMax(a.keys + f, wbest);
    }
    if (prof) {
      prof[2] = p_flag;
      prof[3] = p_grp;
      prof[4] = gtimer();  // chain warps done (the CTA's end)
      prof[5] = p_chain;
    }
  } else if (warp == kMmaWarp) {
    // ===================== MMA issuer (one thread)
    // Straight-line issue: the thread's scalar work per MMA is one 64-bit descriptor add and one
    // TMEM address add (measured: a loop body of ~30 dependent scalar instructions per MMA
    // throttles issue to ~250 cycles per MMA, ~4x the tensor pipe's time for N = 136).
    {  // the whole warp runs the loop (warp-uniform operands -> uniform datapath); one lane issues
      const uint32_t bhi = smem_u32(smem_tc);
      const uint64_t dlo_off = (uint64_t)(((uint32_t)npl * plane) >> 4);  // hi -> lo operand (descriptor units)
      constexpr uint64_t kKStep = (uint64_t)((2 * plane_bytes()) >> 4);   // one K-step of 16 = two planes of 8
      int b = 0, ph = 0, ch = 0, s = 0, g = 0, nrel_done = 0;
      (void)ch;
      // Window trimming: the window of group g holds output rows u = kG g - kHB + 1 + c
      // (c < kNWin); only 0 <= u < nu are kept, so during the ramp-in / ramp-out rows of the
      // CTA (the first and last kHB - 1 image rows) the MMAs cover just the columns [c0, c0+nN)
      // holding valid rows (8-column granularity, N >= 16).  The skipped columns belong to rows
      // that are never drained, so the accumulated values of the kept rows are unchanged.
      int c0 = 0, nN = kNWin;
      auto trim = [&](int gg) {
        const int lo = max(0, kHB - 1 - kG * gg);
        const int chi = min(kNWin, nu + kHB - 1 - kG * gg);
        c0 = (lo / 8) * 8;
        nN = ((chi - c0 + 7) / 8) * 8;
        if (nN < 16) {
          nN = 16;
          if (c0 + 16 > kNWin) c0 = kNWin - 16;
        }
        if (TC_EXP(4096)) { c0 = 0; nN = kNWin; }
      };
      // Software-pipelined issue: the wait for stage q+1's operand happens while the last K-step
      // of stage q is still queued (the tensor pipe's queue is short; a per-stage wait between
      // the last MMA of q and the first of q+1 left it idle for a few hundred cycles per stage).
      // Per stage the issuer only adds constants to precomputed uniform operands: barrier
      // addresses are converted once, the B descriptor moves by one 16-byte row per image row,
      // the accumulator column / instruction descriptor change once per group.
      const uint32_t full0 = smem_u32(&a_full[0]), done0 = smem_u32(&mma_done[0]);
      const uint32_t gdone0 = smem_u32(&grp_done[0]), drained0 = smem_u32(&drained[0]);
      unsigned long long* mprof = (a.exp & 32) && lane == 0 ? a.prof + (int64_t)tk * 8 : nullptr;
      unsigned long long m_drained = 0, m_afull = 0;
      if (mprof) mprof[0] = gtimer();
      const bool leader = elect_one();
      int q = 0;
      if (nch == 1 && !TC_EXP(262144) && !TC_EXP(1048576)) {
        // One template column chunk per image row (WC = 32, the default): per stage the warp waits
        // for its operand (one try_wait that falls through when the producers are ahead, as they
        // normally are), then the elected lane issues the stage's 6 MMAs and the commit with
        // nothing in between.  The tensor pipe queues only about one MMA, so the scalar work between
        // two MMAs must stay short: the earlier form (the operand wait between the two K-steps, the
        // unrolled 30-try wait loops whose success path was a taken branch) ran at ~135 cycles per
        // N = 136 MMA; the pipe's rate is 68 (tools/microbench/issue_probe.cu, tc_trace.cu).
        uint32_t phs = 0;
#pragma unroll 1
        for (g = 0; q < nstage; ++g) {
          const uint32_t col = (uint32_t)((g * kG) % kRelocAt);
          if (col == 0 && g > 0 && !TC_EXP(2048)) {  // window restart: relocate the live columns first
            const int qp = q - 1;   // MMAs complete in order: the last stage's completion covers all
            mbar_wait_u32(done0 + 8 * (qp % kNBuf), (uint32_t)((qp / kNBuf) & 1));
            fence_after();
            fence_before();
            if (leader) mbar_arrive(&reloc_req);
            __syncwarp();
            mbar_wait_bounded(&reloc_done, (uint32_t)(nrel_done & 1));
            fence_after();
            ++nrel_done;
          }
          if (lane == 0) TC_STAMP(6, g);
          if (g >= kGRing) {  // the window's newest columns were drained (and zeroed) after group g - kGRing
            const unsigned long long t0 = mprof ? gtimer() : 0ull;
            if (!TC_EXP(16)) mbar_wait_fall(drained0 + 8 * ((g - kGRing) % kGRing), (uint32_t)(((g - kGRing) / kGRing) & 1));
            if (mprof) m_drained += gtimer() - t0;
            fence_after();
          }
          if (lane == 0) TC_STAMP(7, g);
          trim(g);
          const uint32_t dcol = tbase + col + (uint32_t)c0;
          const uint32_t id = idesc_bf16(nN);
          const uint64_t dg = sdesc(bhi + (uint32_t)(kG - 1 + c0) * 16, plane, 128);
          // stages in pairs (b even: q = 8 g and kNBuf = 6 are even; the pair shares its phase)
#pragma unroll 1
          for (int st = 0; st < kG; st += 2, q += 2) {
            if (!TC_EXP(16)) {
              mbar_wait_fall(full0 + 8 * b, phs);
              mbar_wait_fall(full0 + 8 * (b + 1), phs);
            }
            fence_after();
            if (lane == 0) {
              TC_STAMP(3, q);
              TC_STAMP(3, q + 1);
            }
            const uint32_t ah = tbase + a_col0 + (uint32_t)(b * kWB), ah1 = ah + kWB;
            const uint64_t dh = dg - (uint64_t)st, dh1 = dh - 1;
            if (leader) {
              mma_bf16(dcol, ah, dh, id);
              mma_bf16(dcol, ah, dh + dlo_off, id);
              mma_bf16(dcol, ah + kWB / 2, dh, id);
              mma_bf16(dcol, ah + 8, dh + kKStep, id);
              mma_bf16(dcol, ah + 8, dh + dlo_off + kKStep, id);
              mma_bf16(dcol, ah + kWB / 2 + 8, dh + kKStep, id);
              commit_u32(done0 + 8 * b);
              mma_bf16(dcol, ah1, dh1, id);
              mma_bf16(dcol, ah1, dh1 + dlo_off, id);
              mma_bf16(dcol, ah1 + kWB / 2, dh1, id);
              mma_bf16(dcol, ah1 + 8, dh1 + kKStep, id);
              mma_bf16(dcol, ah1 + 8, dh1 + dlo_off + kKStep, id);
              mma_bf16(dcol, ah1 + kWB / 2 + 8, dh1 + kKStep, id);
              commit_u32(done0 + 8 * (b + 1));
            }
            __syncwarp();
            if (lane == 0) {
              TC_STAMP(4, q);
              TC_STAMP(4, q + 1);
            }
            b += 2;
            if (b == kNBuf) {
              b = 0;
              phs ^= 1u;
            }
          }
          if (leader) commit_u32(gdone0 + 8 * (g % kGRing));  // group g's MMAs complete -> epilogue drains it
          __syncwarp();
          if (mprof && tk < 4 && g < 64) a.prof[(int64_t)gridDim.x * gridDim.y * 8 + 256 + tk * 64 + g] = gtimer();
        }
        q = nstage;
      }
      if (TC_EXP(262144)) {  // trace experiment: the issue_probe loop (fixed operands) inside this kernel
        for (int it = 0; it < nstage; ++it) {
          const int ss = it & 7, bb = it % 6;
          uint32_t dc = tbase + (uint32_t)(((it >> 3) * 8) % 176);
          uint32_t id = idesc_bf16(kNWin);
          uint64_t dg = sdesc(bhi + (uint32_t)(kG - 1) * 16, plane, 128);
          if (TC_EXP(524288)) {  // + the real window trimming and D column of the stage's group
            trim(it >> 3);
            dc = tbase + (uint32_t)(((it >> 3) * kG) % kRelocAt) + (uint32_t)c0;
            id = idesc_bf16(nN);
            dg = sdesc(bhi + (uint32_t)(kG - 1 + c0) * 16, plane, 128);
          }
          const uint32_t ah = tbase + a_col0 + (uint32_t)(bb * kWB);
          if (lane == 0) TC_STAMP(3, it);
          if (leader) {
#pragma unroll
            for (int kk = 0; kk < 2; ++kk) {
              mma_bf16(dc, ah + kk * 8, dg - (uint64_t)ss + kk * kKStep, id);
              mma_bf16(dc, ah + kk * 8, dg - (uint64_t)ss + dlo_off + kk * kKStep, id);
              mma_bf16(dc, ah + kWB / 2 + kk * 8, dg - (uint64_t)ss + kk * kKStep, id);
            }
            commit_u32(done0 + 8 * bb);
          }
          __syncwarp();
        }
        q = nstage;
      }
#pragma unroll 1
      for (g = 0; q < nstage; ++g) {
        const uint32_t col = (uint32_t)((g * kG) % kRelocAt);
        if (!TC_EXP(2048) && col == 0 && g > 0) {  // window restart: relocate the live columns first
          const int qp = q - 1;  // MMAs complete in order: the last stage's completion covers all
          mbar_wait_u32(done0 + 8 * (qp % kNBuf), (uint32_t)((qp / kNBuf) & 1));
          fence_after();
          fence_before();
          if (leader) mbar_arrive(&reloc_req);
          __syncwarp();
          mbar_wait_bounded(&reloc_done, (uint32_t)(nrel_done & 1));
          fence_after();
          ++nrel_done;
        }
        if (g >= kGRing && !TC_EXP(16)) {  // the window's newest columns were drained (and zeroed) after group g - kGRing
          const unsigned long long t0 = mprof ? gtimer() : 0ull;
          const uint32_t dr = drained0 + 8 * ((g - kGRing) % kGRing), dp = (uint32_t)(((g - kGRing) / kGRing) & 1);
          if (!mbar_try_u32(dr, dp)) mbar_wait_u32(dr, dp);
          if (mprof) m_drained += gtimer() - t0;
          fence_after();
        }
        trim(g);
        const uint32_t dcol = tbase + col + (uint32_t)c0;
        const uint32_t id = idesc_bf16(nN);
        // B window of (s = 0, ch = 0): row kG - 1 + c0 of the reversed block
        const uint64_t dg = sdesc(bhi + (uint32_t)(kG - 1 + c0) * 16, plane, 128);
        // Stages in pairs: both operands' waits first (the producers run several stages ahead, so
        // both normally succeed at the first try and fall through), then 12 MMAs in straight-line
        // code.  The tensor pipe queues about one MMA: any branch or dependent scalar latency
        // between two MMAs is lost tensor time (tools/microbench/issue_probe.cu: 6 MMAs per stage
        // with a wait and the loop's branches between them cost ~135 cycles per MMA; straight-line
        // MMAs run at the pipe's rate, 68 cycles at N = 136).
        const int qend = q + kG * nch;  // nstage is a whole number of groups; kG * nch is even
        int s0 = 0, c0h = 0;            // (image row in group, column chunk) of stage q
#pragma unroll 1
        for (; q < qend; q += 2) {
          const int s1 = c0h + 1 < nch ? s0 : s0 + 1, c1 = c0h + 1 < nch ? c0h + 1 : 0;
          const int b1 = b + 1;  // b is even: the pair shares the phase
          if (!TC_EXP(16)) {
            const unsigned long long t0 = mprof ? gtimer() : 0ull;
            if (!mbar_try_u32(full0 + 8 * b, (uint32_t)ph)) mbar_wait_u32(full0 + 8 * b, (uint32_t)ph);
            if (!mbar_try_u32(full0 + 8 * b1, (uint32_t)ph)) mbar_wait_u32(full0 + 8 * b1, (uint32_t)ph);
            if (mprof) m_afull += gtimer() - t0;
          }
          if (!TC_EXP(16384)) fence_after();
          if (lane == 0) {
            TC_STAMP(3, q);
            TC_STAMP(3, q + 1);
          }
          const uint64_t dh0 = dg - (uint64_t)s0 + (uint64_t)(((uint32_t)c0h * (kWB / 8) * plane) >> 4);
          const uint64_t dh1 = dg - (uint64_t)s1 + (uint64_t)(((uint32_t)c1 * (kWB / 8) * plane) >> 4);
          const uint32_t ah0 = tbase + a_col0 + (uint32_t)(b * kWB), ah1 = ah0 + kWB;
          if (leader) {
#pragma unroll
            for (int kk = 0; kk < kWB / 16; ++kk) {
              mma_bf16(dcol, ah0 + kk * 8, dh0 + kk * kKStep, id);
              mma_bf16(dcol, ah0 + kk * 8, dh0 + dlo_off + kk * kKStep, id);
              mma_bf16(dcol, ah0 + kWB / 2 + kk * 8, dh0 + kk * kKStep, id);
            }
            commit_u32(done0 + 8 * b);
#pragma unroll
            for (int kk = 0; kk < kWB / 16; ++kk) {
              mma_bf16(dcol, ah1 + kk * 8, dh1 + kk * kKStep, id);
              mma_bf16(dcol, ah1 + kk * 8, dh1 + dlo_off + kk * kKStep, id);
              mma_bf16(dcol, ah1 + kWB / 2 + kk * 8, dh1 + kk * kKStep, id);
            }
            commit_u32(done0 + 8 * b1);
          }
          __syncwarp();
          if (lane == 0) {
            TC_STAMP(4, q);
            TC_STAMP(4, q + 1);
          }
          b += 2;
          if (b == kNBuf) {
            b = 0;
            ph ^= 1;
          }
          s0 = c1 + 1 < nch ? s1 : s1 + 1;
          c0h = c1 + 1 < nch ? c1 + 1 : 0;
        }
        if (leader) commit_u32(gdone0 + 8 * (g % kGRing));  // group g's MMAs complete -> epilogue drains it
        __syncwarp();
        if (mprof && tk < 4 && g < 64) a.prof[(int64_t)gridDim.x * gridDim.y * 8 + 256 + tk * 64 + g] = gtimer();
      }
      if (mprof) {
        mprof[1] = gtimer();
        mprof[6] = m_drained;
        mprof[7] = m_afull;
      }
    }
    __syncwarp();
  }
  fence_before();
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tbase));
}

// Image operand of the tensor-core numerator: every element of the band's rows split once into
// x = hi + lo (hi = bf16(x), lo = bf16(x - hi), both round-to-nearest), then stored in the layout the
// producer warps copy into TMEM without any per-element work: with P_k = (hi_k | hi_{k+1} << 16) and
// Q_k = (lo_k | lo_{k+1} << 16) (zero past the row end), row r holds two planes of 8-byte elements,
// E_k = (P_k, P_{k+2}) then F_k = (Q_k, Q_{k+2}), k < wp = W rounded up to even (16-byte TMA
// strides): [batch][rows][2][wp] x 8 bytes (16 bytes per image element).  grid = (ceil(wp/4/128),
// rows, batch), block = 128, 4 elements per thread.  out row r = image row row0 + r.
// With `ts` (centred operand): every element is first shifted by the template mean,
// x = I - tc_center(ts, n) (fp32), so the accumulators hold sum A_C (I - c) -- sums without the
// image's DC level -- and the epilogue adds c * sum A_C back (exact: tc_center is the same fp32
// value there).  ts = nullptr: the raw image.
__global__ void __launch_bounds__(128) tm_tc_split(const float* __restrict__ img, int64_t pitch, int64_t frame_stride,
                                                   int W, int row0, uint2* __restrict__ out, int64_t out_frame_stride,
                                                   int wp, const TemplateStats* ts, double n) {
  const int c = (blockIdx.x * 128 + threadIdx.x) * 4;
  const float cen = tc_center(ts, n);
  const int r = blockIdx.y, f = blockIdx.z;
  const float* src = img + (int64_t)f * frame_stride + (int64_t)(row0 + r) * pitch;
  // elements c .. c + 3 (one 16-byte load when aligned); c + 4 .. c + 6 from the next lane
  float x[4];
  if (c + 4 <= W && ((reinterpret_cast<uintptr_t>(src + c) & 15) == 0)) {
    const float4 v = __ldg(reinterpret_cast<const float4*>(src + c));
    x[0] = v.x; x[1] = v.y; x[2] = v.z; x[3] = v.w;
  } else {
#pragma unroll
    for (int k = 0; k < 4; ++k) x[k] = c + k < W ? __ldg(src + c + k) : 0.0f;
  }
  uint32_t h[7], l[7];
#pragma unroll
  for (int k = 0; k < 4; ++k) {
    const uint32_t s2 = tc::split_bf16(c + k < W ? x[k] - cen : 0.0f);
    h[k] = s2 & 0xffffu;
    l[k] = s2 >> 16;
  }
  const int lane = threadIdx.x & 31;
#pragma unroll
  for (int k = 0; k < 3; ++k) {
    uint32_t hn = __shfl_down_sync(0xffffffffu, h[k], 1), ln = __shfl_down_sync(0xffffffffu, l[k], 1);
    if (lane == 31) {  // the warp's last lane: its neighbour's elements directly
      const uint32_t s2 = tc::split_bf16(c + 4 + k < W ? __ldg(src + c + 4 + k) - cen : 0.0f);
      hn = s2 & 0xffffu;
      ln = s2 >> 16;
    }
    h[4 + k] = hn;
    l[4 + k] = ln;
  }
  if (c >= wp) return;
  uint32_t P[6], Q[6];
#pragma unroll
  for (int k = 0; k < 6; ++k) {
    P[k] = h[k] | (h[k + 1] << 16);
    Q[k] = l[k] | (l[k + 1] << 16);
  }
  uint2* dst = out + (int64_t)f * out_frame_stride + (int64_t)r * 2 * wp + c;
  if (c + 4 <= wp) {  // wp is even and c a multiple of 4: 16-byte aligned pairs of elements
    reinterpret_cast<uint4*>(dst)[0] = make_uint4(P[0], P[2], P[1], P[3]);
    reinterpret_cast<uint4*>(dst)[1] = make_uint4(P[2], P[4], P[3], P[5]);
    reinterpret_cast<uint4*>(dst + wp)[0] = make_uint4(Q[0], Q[2], Q[1], Q[3]);
    reinterpret_cast<uint4*>(dst + wp)[1] = make_uint4(Q[2], Q[4], Q[3], Q[5]);
  } else {
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      if (c + k < wp) {
        dst[k] = make_uint2(P[k], P[k + 2]);
        dst[wp + k] = make_uint2(Q[k], Q[k + 2]);
      }
    }
  }
}

// Numerator of the last V - v_lo (< 128) output columns, which would otherwise cost a whole
// column of tensor-core CTAs (V = W - w + 1 is 1 mod 128 for power-of-two frames and
// templates): one warp per (frame, output row, column); lanes split the template columns, a
// fresh fp32 partial per template row, then a warp sum: the full numerator, written to the
// running-numerator plane (normalised by tm_tc_tail).  Loads of RB template
// rows are issued before their products (the kernel is load-latency bound).  grid =
// ceil(items / 8), block = 256.
template <int JC>  // JC = ceil(w / 32) template columns per lane
__global__ void __launch_bounds__(256) tm_tc_cols(const float* __restrict__ img, int64_t pitch, int64_t frame_stride,
                                                  const float* __restrict__ tplC, int tplP, int h, int w, int v_lo,
                                                  int V, int u_begin, int Ub, int batch, float* __restrict__ acc,
                                                  int64_t acc_frame_stride) {
  const int nc = V - v_lo;
  const int64_t item = (int64_t)blockIdx.x * 8 + (threadIdx.x >> 5);
  if (item >= (int64_t)batch * Ub * nc) return;
  const int lane = threadIdx.x & 31;
  const int c = (int)(item % nc);
  const int64_t t = item / nc;
  const int ur = (int)(t % Ub), f = (int)(t / Ub);
  const float* I = img + (int64_t)f * frame_stride + (int64_t)(u_begin + ur) * pitch + v_lo + c + lane;
  const float* T = tplC + lane;  // zero-padded to tplP >= 32 * JC columns
  constexpr int RB = 8;           // template rows per batch of loads (RB * JC * 2 loads in flight)
  float tot = 0.0f;
  for (int i0 = 0; i0 < h; i0 += RB) {
    float tv[RB][JC], xv[RB][JC];
#pragma unroll
    for (int r = 0; r < RB; ++r)
#pragma unroll
      for (int k = 0; k < JC; ++k) {
        const bool ok = i0 + r < h && lane + 32 * k < w;
        tv[r][k] = ok ? __ldg(T + (int64_t)(i0 + r) * tplP + 32 * k) : 0.0f;
        xv[r][k] = ok ? __ldg(I + (int64_t)(i0 + r) * pitch + 32 * k) : 0.0f;
      }
#pragma unroll
    for (int r = 0; r < RB; ++r) {
      float pr = 0.0f;  // fresh partial per template row
#pragma unroll
      for (int k = 0; k < JC; ++k) pr = fmaf(tv[r][k], xv[r][k], pr);
      tot += pr;
    }
  }
#pragma unroll
  for (int d = 16; d; d >>= 1) tot += __shfl_xor_sync(0xffffffffu, tot, d);
  if (lane == 0) acc[(int64_t)f * acc_frame_stride + (int64_t)ur * V + v_lo + c] = tot;
}

// As tm_tc_cols, RWN consecutive output rows per warp: template row i is loaded once for the
// RWN rows, and the RWN image rows in flight slide down (row ur0 + r + i lives in register slot
// (r + i) mod RWN), so each step loads one template row and one new image row for RWN x 32 JC
// products (0.5 loads per product at RWN = 4, was 2).  Per output the products still come
// row by row with a fresh partial per template row (the tm_tc_cols order).  grid =
// ceil(items / 8) with items = batch x ceil(Ub / RWN) x columns, block = 256.
template <int JC, int RWN>
__global__ void __launch_bounds__(256) tm_tc_cols_rw(const float* __restrict__ img, int64_t pitch,
                                                     int64_t frame_stride, const float* __restrict__ tplC, int tplP,
                                                     int h, int w, int v_lo, int V, int u_begin, int Ub, int batch,
                                                     float* __restrict__ acc, int64_t acc_frame_stride) {
  const int nc = V - v_lo, nrb = (Ub + RWN - 1) / RWN;
  const int64_t item = (int64_t)blockIdx.x * 8 + (threadIdx.x >> 5);
  if (item >= (int64_t)batch * nrb * nc) return;
  const int lane = threadIdx.x & 31;
  const int c = (int)(item % nc);
  const int64_t t = item / nc;
  const int ur0 = (int)(t % nrb) * RWN, f = (int)(t / nrb);
  const int nrows_in = Ub + h - 1;  // band rows + halo (relative to u_begin)
  const float* I = img + (int64_t)f * frame_stride + (int64_t)(u_begin + ur0) * pitch + v_lo + c + lane;
  const float* T = tplC + lane;
  bool okc[JC];
#pragma unroll
  for (int k = 0; k < JC; ++k) okc[k] = lane + 32 * k < w;
  float win[RWN][JC];
  auto load_row = [&](float (&dst)[JC], int rr) {  // image row ur0 + rr of the band
    const bool ok = ur0 + rr < nrows_in;
#pragma unroll
    for (int k = 0; k < JC; ++k) dst[k] = (ok && okc[k]) ? __ldg(I + (int64_t)rr * pitch + 32 * k) : 0.0f;
  };
#pragma unroll
  for (int r = 0; r < RWN - 1; ++r) load_row(win[r], r);
  float tot[RWN];
#pragma unroll
  for (int r = 0; r < RWN; ++r) tot[r] = 0.0f;
  for (int i0 = 0; i0 < h; i0 += RWN) {
#pragma unroll
    for (int s = 0; s < RWN; ++s) {
      const int i = i0 + s;
      if (i < h) {
        load_row(win[(RWN - 1 + s) % RWN], RWN - 1 + i);
        float tv[JC];
#pragma unroll
        for (int k = 0; k < JC; ++k) tv[k] = okc[k] ? __ldg(T + (int64_t)i * tplP + 32 * k) : 0.0f;
#pragma unroll
        for (int r = 0; r < RWN; ++r) {
          float pr = 0.0f;  // fresh partial per template row
#pragma unroll
          for (int k = 0; k < JC; ++k) pr = fmaf(tv[k], win[(r + s) % RWN][k], pr);
          tot[r] += pr;
        }
      }
    }
  }
#pragma unroll
  for (int r = 0; r < RWN; ++r) {
#pragma unroll
    for (int d = 16; d; d >>= 1) tot[r] += __shfl_xor_sync(0xffffffffu, tot[r], d);
  }
  if (lane == 0)
#pragma unroll
    for (int r = 0; r < RWN; ++r)
      if (ur0 + r < Ub) acc[(int64_t)f * acc_frame_stride + (int64_t)(ur0 + r) * V + v_lo + c] = tot[r];
}

// Template operand: for block (bi, bj) the reversed, zero-padded rows Rv[k] = A_C[i0 + K0 - k]
// (K0 = kHB + kG - 2, zero outside the block / template), split into tf32 hi and fp32 lo, laid
// out [2][WC/4 planes][kLB rows][4 floats] (the UMMA K-major no-swizzle canonical layout with
// 16-byte rows).  grid = nblk, block = 256.
__global__ void tm_tc_tpl_prep(const float* __restrict__ tplC, int tplP, int h, int w, int WC, int nbj,
                               float* __restrict__ tcB) {
  using namespace tc;
  const int blk = blockIdx.x, bi = blk / nbj, bj = blk % nbj;
  const int i0 = bi * kHB, j0 = bj * WC;
  const int npl = WC / 8;
  uint16_t* out = reinterpret_cast<uint16_t*>(tcB) + (int64_t)blk * (b_bytes(WC) / 2);
  const int n = npl * kLB * 8;
  for (int e = threadIdx.x; e < n; e += blockDim.x) {
    const int c = e / (kLB * 8), k = (e / 8) % kLB, t = e % 8;
    const int row = kHB + kG - 2 - k;
    const int i = i0 + row, j = j0 + 8 * c + t;
    const float val = (row >= 0 && row < kHB && i < h && j < w) ? tplC[(int64_t)i * tplP + j] : 0.0f;
    const uint32_t hl = split_bf16(val);
    out[e] = (uint16_t)(hl & 0xffffu);
    out[n + e] = (uint16_t)(hl >> 16);
  }
}

constexpr int kPrepSmemFloats = 48 * 1024;  // tm_tc_prep: templates up to 192 KB (else the two-kernel prep)
// Template prep of the tensor-core path in one launch (Fig 5.2, a1, + the MMA operand): every
// CTA forms the template mean (same code, same order: every CTA gets the same value), writes
// its share of the centred, zero-padded template A_C = (float)(T - mean) (HP x WP, read by
// tm_tc_cols) and its own template block's reversed, hi/lo-split operand (as tm_tc_tpl_prep,
// from the same expression); CTA 0 adds A_D = sum (T - mean)^2, the sum of the fp32 A_C values,
// the flat flag and resets the frame keys.  grid = nblk, block = 1024.
__global__ void __launch_bounds__(1024) tm_tc_prep(const float* __restrict__ tmpl, int64_t tpitch, int h, int w,
                                                   float* __restrict__ tplC, int HP, int WP, TemplateStats* ts,
                                                   unsigned long long* keys, int batch, int WC, int nbj,
                                                   float* __restrict__ tcB) {
  using namespace tc;
  extern __shared__ float tsm[];  // the whole template, dense h x w (n <= kPrepSmemFloats)
  __shared__ double red[32];
  {  // several templates (ROI mode): blockIdx.y = template t, rows of the stacked templates
    const int t = blockIdx.y;
    tmpl += (int64_t)t * h * tpitch;
    tplC += (int64_t)t * HP * WP;
    ts += t;
    tcB += (int64_t)t * gridDim.x * (b_bytes(WC) / 4);  // (float units: the byte size / 4)
  }
  const int n = h * w;
  // one pass over the template, staged in shared memory: float4 loads when rows allow it
  // (w, pitch and base 16-byte aligned), all of a thread's loads in flight
  double s = 0.0, s2 = 0.0;
  const bool v4 = (w & 3) == 0 && (tpitch & 3) == 0 && (reinterpret_cast<uintptr_t>(tmpl) & 15) == 0;
  if (v4) {
    const int g4 = w >> 2, n4 = n >> 2;
    constexpr int LB = 4;
    for (int k0 = threadIdx.x; k0 < n4; k0 += LB * blockDim.x) {
      float4 x[LB];
#pragma unroll
      for (int r = 0; r < LB; ++r) {
        const int k = k0 + r * blockDim.x;
        x[r] = k < n4 ? __ldg(reinterpret_cast<const float4*>(tmpl + (int64_t)(k / g4) * tpitch) + k % g4)
                      : make_float4(0.f, 0.f, 0.f, 0.f);
      }
#pragma unroll
      for (int r = 0; r < LB; ++r) {
        const int k = k0 + r * blockDim.x;
        if (k < n4) reinterpret_cast<float4*>(tsm)[k] = x[r];
        s += ((double)x[r].x + (double)x[r].y) + ((double)x[r].z + (double)x[r].w);
        s2 += ((double)x[r].x * x[r].x + (double)x[r].y * x[r].y) + ((double)x[r].z * x[r].z + (double)x[r].w * x[r].w);
      }
    }
  } else {
    constexpr int LB = 8;
    for (int k0 = threadIdx.x; k0 < n; k0 += LB * blockDim.x) {
      float x[LB];
#pragma unroll
      for (int r = 0; r < LB; ++r) {
        const int k = k0 + r * blockDim.x;
        x[r] = k < n ? __ldg(tmpl + (int64_t)(k / w) * tpitch + (k % w)) : 0.0f;
      }
#pragma unroll
      for (int r = 0; r < LB; ++r) {
        const int k = k0 + r * blockDim.x;
        if (k < n) tsm[k] = x[r];
        s += (double)x[r];
        s2 += (double)x[r] * (double)x[r];
      }
    }
  }
  s = block_sum_d(s, red);  // (its barriers also publish tsm)
  s2 = block_sum_d(s2, red);
  const double mean = s / (double)n;
  // centred, zero-padded template (HP x WP), row-strided over the CTAs
  for (int i = blockIdx.x; i < HP; i += gridDim.x)
    for (int j = threadIdx.x; j < WP; j += blockDim.x)
      tplC[(int64_t)i * WP + j] = (i < h && j < w) ? (float)((double)tsm[i * w + j] - mean) : 0.0f;
  {  // this CTA's template block operand (reversed rows, hi / lo planes; as tm_tc_tpl_prep)
    const int blk = blockIdx.x, bi = blk / nbj, bj = blk % nbj;
    const int i0 = bi * kHB, j0 = bj * WC;
    uint16_t* out = reinterpret_cast<uint16_t*>(tcB + (int64_t)blk * (b_bytes(WC) / 4));
    const int nb = (WC / 8) * kLB * 8;
    for (int e = threadIdx.x; e < nb; e += blockDim.x) {
      const int c = e / (kLB * 8), k = (e / 8) % kLB, t = e % 8;
      const int row = kHB + kG - 2 - k;
      const int i = i0 + row, j = j0 + 8 * c + t;
      const float val = (row >= 0 && row < kHB && i < h && j < w) ? (float)((double)tsm[i * w + j] - mean) : 0.0f;
      const uint32_t hl = split_bf16(val);
      out[e] = (uint16_t)(hl & 0xffffu);
      out[nb + e] = (uint16_t)(hl >> 16);
    }
  }
  if (blockIdx.x != 0) return;
  double e = 0.0, cs = 0.0;
  for (int k = threadIdx.x; k < n; k += blockDim.x) {
    const double a = (double)tsm[k] - mean;
    e += a * a;
    cs += (double)(float)a;
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
  for (int f = threadIdx.x; f < batch; f += blockDim.x) keys[(int64_t)f * gridDim.y + blockIdx.y] = 0ull;
}

// Ragged last columns [v_lo, V) (computed by tm_tc_cols into the running-numerator plane):
// normalise (or SSD), optional surface store, fold into the per-frame argmax keys; the last CTA
// to finish turns every frame's key into its peak (tm_finalize fused) -- the tensor-core kernel
// folded its own columns' keys before this launch (stream order).  grid = max(1, ceil(items /
// 256)), items = batch x Ub x (V - v_lo); block = 256.
__global__ void __launch_bounds__(256) tm_tc_tail(const float* __restrict__ acc, int64_t acc_frame_stride,
                                                  const float* __restrict__ rsv, const float* __restrict__ mean,
                                                  const double* __restrict__ S1, const double* __restrict__ S2,
                                                  int64_t stat_frame_stride, const TemplateStats* tst, int h, int w,
                                                  int V, int v_lo, int u_begin, int Ub, int batch, float* scores,
                                                  int64_t score_frame_stride, unsigned long long* keys, int ssd,
                                                  unsigned int* __restrict__ done, PeakOut* __restrict__ peaks) {
  __shared__ bool last;
  const TemplateStats ts = tst[0];
  const int nc = V - v_lo;
  const int64_t items = (int64_t)batch * Ub * nc;
  const int64_t it = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const double inv_n = 1.0 / ((double)h * (double)w);
  int f = -1;
  unsigned long long key = 0ull;
  if (it < items) {
    const int c = (int)(it % nc);
    const int64_t t = it / nc;
    const int ur = (int)(t % Ub);
    f = (int)(t / Ub);
    const int v = v_lo + c;
    const int64_t o = (int64_t)ur * V + v;
    const float num = acc[(int64_t)f * acc_frame_stride + o];
    float sc;
    if (ssd) {
      const double s1 = S1[(int64_t)f * stat_frame_stride + o], s2 = S2[(int64_t)f * stat_frame_stride + o];
      sc = (float)(ts.sumsq - 2.0 * ((double)num + ts.sum * inv_n * s1) + s2);
    } else {  // the fp32-factor form of tm_tc_finish / the chain epilogue (bitwise the same scores)
      const float rse = ts.flat ? 0.0f : (float)(1.0 / sqrt(ts.energy));
      const float r = fmaf(-(float)ts.csum, mean[(int64_t)f * stat_frame_stride + o], num) *
                      (rsv[(int64_t)f * stat_frame_stride + o] * rse);
      sc = r > 1.0f ? 1.0f : (r < -1.0f ? -1.0f : r);
    }
    if (scores) scores[(int64_t)f * score_frame_stride + o] = sc;
    key = make_key(ssd ? -sc : sc, (uint32_t)((int64_t)(u_begin + ur) * V + v));
  }
  // a warp whose items all belong to one frame folds them first (the usual case)
  const int f0 = __shfl_sync(0xffffffffu, f, 0);
  if (__all_sync(0xffffffffu, f == f0)) {
    key = warp_max_key(key);
    if ((threadIdx.x & 31) == 0 && f0 >= 0 && key > __ldcg(keys + f0)) atomicMax(keys + f0, key);
  } else if (f >= 0 && key > __ldcg(keys + f)) {
    atomicMax(keys + f, key);
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    last = atomicAdd(done, 1u) == gridDim.x - 1;
  }
  __syncthreads();
  if (!last) return;
  __threadfence();
  for (int fr = threadIdx.x; fr < batch; fr += blockDim.x) {
    const unsigned long long k = atomicOr(keys + fr, 0ull);
    const uint32_t idx = key_index(k);
    PeakOut pk;
    pk.score = ssd ? -key_score(k) : key_score(k);
    pk.u = (int32_t)(idx / (uint32_t)V);
    pk.v = (int32_t)(idx % (uint32_t)V);
    pk.flags = (ts.flat && !ssd) ? (kFlatTemplate | kInvalid) : 0u;
    peaks[fr] = pk;
  }
  if (threadIdx.x == 0) *done = 0u;  // ready for the next call (stream-ordered)
}

// Planes mode (few template blocks): sum the blocks' partial numerators in block order, normalise
// (NCC from the window kernels' fp32 factors, |error| <= ~3e-7; SSD from the fp64 sums), optional
// surface store, per-frame argmax keys; the last CTA writes every frame's peak.  Columns >= v_cols
// (the ragged last columns, tm_tc_cols) hold their full numerator in block 0's plane.
// grid = (ceil(V / (256 kFinV)), ceil(Ub / kFinR), batch), block = 256.
constexpr int kFinV = 4;
constexpr int kFinR = 2;  // output rows per CTA (half the CTAs, and half the same-address atomics, of one row each)
__global__ void __launch_bounds__(256) tm_tc_finish(const float* __restrict__ part, int nblk, int64_t blk_stride,
                                                    int64_t frame_stride, const float* __restrict__ rsv,
                                                    const float* __restrict__ mean, const double* __restrict__ S1,
                                                    const double* __restrict__ S2, int64_t stat_frame_stride,
                                                    const TemplateStats* tst, int h, int w, int V, int v_cols,
                                                    int u_begin, float* scores, int64_t score_frame_stride,
                                                    unsigned long long* keys, int ssd, unsigned int* __restrict__ done,
                                                    PeakOut* __restrict__ peaks, int batch, int Ub) {
  __shared__ unsigned long long red[32];
  __shared__ bool last;
  const int f = blockIdx.z;
  const TemplateStats ts = tst[0];
  const double inv_n = 1.0 / ((double)h * (double)w);
  const float csf = (float)ts.csum, rse = ts.flat ? 0.0f : (float)(1.0 / sqrt(ts.energy));
  unsigned long long best = 0ull;
  const int vb = blockIdx.x * 256 * kFinV + threadIdx.x;
  // every row's loads in flight at once (planes mode has at most 8 blocks), then the block-order
  // sum ((p0 + p1) + p2) + ... per output (the kernel is load-latency bound)
  float tot[kFinR][kFinV], fa[kFinR][kFinV], fb[kFinR][kFinV];
#pragma unroll
  for (int rr = 0; rr < kFinR; ++rr) {
    const int ur = blockIdx.y * kFinR + rr;
    const int64_t so = (int64_t)f * stat_frame_stride + (int64_t)ur * V;
#pragma unroll
    for (int k = 0; k < kFinV; ++k) {
      const int v = vb + k * 256;
      tot[rr][k] = 0.0f;
      fa[rr][k] = fb[rr][k] = 0.0f;
      if (ur < Ub && v < V && !ssd) {
        fa[rr][k] = __ldg(rsv + so + v);
        fb[rr][k] = __ldg(mean + so + v);
      }
    }
  }
  for (int b0 = 0; b0 < nblk; b0 += 4) {
    float x[kFinR][4][kFinV];
#pragma unroll
    for (int rr = 0; rr < kFinR; ++rr) {
      const int ur = blockIdx.y * kFinR + rr;
      const int64_t ro = (int64_t)f * frame_stride + (int64_t)ur * V;
#pragma unroll
      for (int bb = 0; bb < 4; ++bb)
#pragma unroll
        for (int k = 0; k < kFinV; ++k) {
          const int v = vb + k * 256, b = b0 + bb;
          x[rr][bb][k] = (ur < Ub && b < nblk && v < V && (b == 0 || v < v_cols))
                             ? __ldcg(part + (int64_t)b * blk_stride + ro + v)
                             : 0.0f;
        }
    }
#pragma unroll
    for (int rr = 0; rr < kFinR; ++rr)
#pragma unroll
      for (int bb = 0; bb < 4; ++bb)
#pragma unroll
        for (int k = 0; k < kFinV; ++k)
          if (b0 + bb < nblk) tot[rr][k] = (b0 + bb == 0) ? x[rr][bb][k] : tot[rr][k] + x[rr][bb][k];
  }
#pragma unroll
  for (int rr = 0; rr < kFinR; ++rr) {
    const int ur = blockIdx.y * kFinR + rr;
    if (ur >= Ub) break;
    const int u = u_begin + ur;
    const int64_t so = (int64_t)f * stat_frame_stride + (int64_t)ur * V;
#pragma unroll
    for (int k = 0; k < kFinV; ++k) {
      const int v = vb + k * 256;
      if (v >= V) break;
      float sc;
      if (ssd) {
        sc = (float)(ts.sumsq - 2.0 * ((double)tot[rr][k] + ts.sum * inv_n * __ldg(S1 + so + v)) + __ldg(S2 + so + v));
      } else {
        const float r = fmaf(-csf, fb[rr][k], tot[rr][k]) * (fa[rr][k] * rse);
        sc = r > 1.0f ? 1.0f : (r < -1.0f ? -1.0f : r);
      }
      if (scores) scores[(int64_t)f * score_frame_stride + (int64_t)ur * V + v] = sc;
      const unsigned long long key = make_key(ssd ? -sc : sc, (uint32_t)((int64_t)u * V + v));
      best = key > best ? key : best;
    }
  }
  best = block_max_key(best, red);
  if (threadIdx.x == 0) {
    if (best && best > __ldcg(keys + f)) atomicMax(keys + f, best);
    __threadfence();
    last = atomicAdd(done, 1u) == gridDim.x * gridDim.y * gridDim.z - 1;
  }
  __syncthreads();
  if (!last) return;
  __threadfence();
  for (int fr = threadIdx.x; fr < batch; fr += blockDim.x) {
    const unsigned long long k = atomicOr(keys + fr, 0ull);
    const uint32_t idx = key_index(k);
    PeakOut pk;
    pk.score = ssd ? -key_score(k) : key_score(k);
    pk.u = (int32_t)(idx / (uint32_t)V);
    pk.v = (int32_t)(idx % (uint32_t)V);
    pk.flags = (ts.flat && !ssd) ? (kFlatTemplate | kInvalid) : 0u;
    peaks[fr] = pk;
  }
  if (threadIdx.x == 0) *done = 0u;  // ready for the next call (stream-ordered)
}

// ROI mode (planes): per (frame, template) sub-problem sp, sum the blocks' partial numerators of
// its clipped ROI in block order, normalise with the template's statistics and the frame's window
// factors, surface [sp][roi_h][roi_w] (clipped positions 0), keys[sp]; the last CTA writes every
// sub-problem's peak.  grid = (ceil(roi_w / (256 kFinV)), roi_h, F T), block = 256.
__global__ void __launch_bounds__(256) tm_tc_finish_roi(const float* __restrict__ part, int nblk,
                                                        int64_t blk_stride, const int32_t* __restrict__ rois,
                                                        int n_tmpl, int roi_h, int roi_w, int U, int V,
                                                        const float* __restrict__ rsv, const float* __restrict__ mean,
                                                        const double* __restrict__ S1, const double* __restrict__ S2,
                                                        int64_t stat_frame_stride, const TemplateStats* tst, int h,
                                                        int w, float* scores, unsigned long long* keys, int ssd,
                                                        unsigned int* __restrict__ done, PeakOut* __restrict__ peaks,
                                                        int nsub) {
  __shared__ unsigned long long red[32];
  __shared__ bool last;
  const int r = blockIdx.y, sp = blockIdx.z;
  const int frm = sp / n_tmpl, tt = sp % n_tmpl;
  const int ru0 = min(max(rois[2 * sp], 0), U - 1), rv0 = min(max(rois[2 * sp + 1], 0), V - 1);
  const int uend = min(ru0 + roi_h, U), vend = min(rv0 + roi_w, V);
  const int u = ru0 + r;
  const TemplateStats ts = tst[tt];
  const double inv_n = 1.0 / ((double)h * (double)w);
  const float csf = (float)ts.csum, rse = ts.flat ? 0.0f : (float)(1.0 / sqrt(ts.energy));
  const int64_t ro = (int64_t)sp * roi_h * roi_w + (int64_t)r * roi_w;
  unsigned long long best = 0ull;
#pragma unroll
  for (int k = 0; k < kFinV; ++k) {
    const int c = blockIdx.x * 256 * kFinV + threadIdx.x + k * 256;
    if (c >= roi_w) break;
    const int v = rv0 + c;
    float sc = 0.0f;
    if (u < uend && v < vend) {
      float tot = 0.0f;
      for (int b = 0; b < nblk; ++b) {  // block order: ((p0 + p1) + p2) + ...
        const float x = __ldcg(part + (int64_t)b * blk_stride + ro + c);
        tot = b == 0 ? x : tot + x;
      }
      const int64_t so = (int64_t)frm * stat_frame_stride + (int64_t)u * V + v;
      if (ssd) {
        sc = (float)(ts.sumsq - 2.0 * ((double)tot + ts.sum * inv_n * __ldg(S1 + so)) + __ldg(S2 + so));
      } else {
        const float q = fmaf(-csf, __ldg(mean + so), tot) * (__ldg(rsv + so) * rse);
        sc = q > 1.0f ? 1.0f : (q < -1.0f ? -1.0f : q);
      }
      const unsigned long long key = make_key(ssd ? -sc : sc, (uint32_t)((int64_t)u * V + v));
      best = key > best ? key : best;
    }
    if (scores) scores[ro + c] = sc;
  }
  best = block_max_key(best, red);
  if (threadIdx.x == 0) {
    if (best && best > __ldcg(keys + sp)) atomicMax(keys + sp, best);
    __threadfence();
    last = atomicAdd(done, 1u) == gridDim.x * gridDim.y * gridDim.z - 1;
  }
  __syncthreads();
  if (!last) return;
  __threadfence();
  for (int q = threadIdx.x; q < nsub; q += blockDim.x) {
    const unsigned long long k = atomicOr(keys + q, 0ull);
    const uint32_t idx = key_index(k);
    const TemplateStats tq = tst[q % n_tmpl];
    PeakOut pk;
    pk.score = ssd ? -key_score(k) : key_score(k);
    pk.u = (int32_t)(idx / (uint32_t)V);
    pk.v = (int32_t)(idx % (uint32_t)V);
    pk.flags = (tq.flat && !ssd) ? (kFlatTemplate | kInvalid) : 0u;
    peaks[q] = pk;
  }
  if (threadIdx.x == 0) *done = 0u;
}

}  // namespace nccb
