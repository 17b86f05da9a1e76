/*
 * ncc.h -- C ABI of the B200-native spatial-domain normalized cross-correlation (NCC)
 * hot path: template matching (TM) and particle image velocimetry (PIV).
 *
 * Paper: N. Moore, "Kernel Specialization for Improved Adaptability and Performance on
 * GPUs" (dissertation / IPDPS-W 2013), /root/reference/PAPER.md, cited as P:<lines>.
 *
 *  - TM computes corr2(template, window) at every valid shift (Listing 5.1 caption
 *    P:250-251, Tab 5.1 caption P:190-191) -- the Pearson coefficient with A-bar, B-bar the
 *    matrix averages (Fig 5.1 caption P:132-137), in the staged form of Fig 5.2:
 *    A_C = template minus its average, A_D = the template's denominator term, B-bar the
 *    window average; numerator stage Fig 5.3.
 *  - PIV correlates each mask (interrogation window of frame A) against the shifted
 *    windows of frame B over a search range (Figs 5.8-5.12 captions P:164-171) and
 *    reports the peak with a 3-point sub-pixel fit (DESIGN.md readings).
 *  - The plan lifecycle follows GPU-PF's specification -> refresh -> execution split
 *    (P:1396-1409): ncc_plan_create validates, selects the specialised kernel variant and
 *    allocates all scratch; the execute calls allocate nothing (except the optional host
 *    staging buffers of the *_host calls, allocated on their first use).
 *
 * Conventions (all entry points):
 *  - Images are row-major fp32.  Frame k of a batch starts at base + k*image_h*image_pitch
 *    (elements).  image_pitch >= image_w.  Device pointers must be 4-byte aligned.
 *  - Ownership: the caller owns every data buffer; the plan owns its scratch, events and
 *    staging buffers.  One plan is used by one stream at a time.
 *  - Execute calls are asynchronous on `stream` (cudaStream_t passed as void*; NULL = the
 *    legacy default stream).  Results are valid after the stream is synchronised.
 *  - Execute calls replay CUDA graphs: the first call with a given set of pointer arguments
 *    captures the plan's launch sequence (on a plan-owned capture stream) and later calls with
 *    the same pointers launch it as one graph; a plan keeps up to 4 such graphs.  Buffers may
 *    be reused or replaced freely between calls (a new pointer set is captured on first use);
 *    NCC_NO_GRAPH=1 in the environment launches kernel by kernel.
 *  - Errors: shape/argument errors are returned by ncc_plan_create
 *    (NCC_ERR_INVALID_ARGUMENT); launch failures by the execute call (NCC_ERR_CUDA).
 *    Data-dependent conditions are never status codes: they are flag bits in the outputs.
 *  - The library never falls back to the CPU.
 */
#ifndef NCC_B200_H
#define NCC_B200_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct ncc_plan_s* ncc_plan;

typedef enum {
    NCC_OK = 0,
    NCC_ERR_INVALID_ARGUMENT = 1, /* bad sizes / pointers / ranges                        */
    NCC_ERR_UNSUPPORTED = 2,      /* valid problem this build cannot run (smem limits)     */
    NCC_ERR_OUT_OF_MEMORY = 3,    /* scratch allocation failed                             */
    NCC_ERR_CUDA = 4,             /* CUDA runtime / launch error (see ncc_last_cuda_error) */
    NCC_ERR_COMPILE = 5,          /* run-time specialisation failed                        */
    NCC_ERR_WRONG_MODE = 6        /* ncc_match on a PIV plan or piv_correlate on a TM plan */
} ncc_status;

enum { NCC_MODE_MATCH = 0, NCC_MODE_PIV = 1 };
/* Score.  NCC: corr2 (Fig 5.1), peak = argmax.  SSD: sum (T - W)^2, the paper's own PIV
 * similarity score (Fig 5.10 caption), peak = argmin (tie -> smallest index);
 * computed from the same numerator as sum T^2 - 2 (sum A_C W + Tbar S1) + S2; PIV sub-pixel
 * for SSD is the 3-point parabola through the minimum; no flat-template flags for SSD.
 * SAD: sum |T - W|, the metric the paper's specialisation example swaps for SSD (Ch. 4,
 * P:1176-1179); peak = argmin, PIV sub-pixel as SSD; computed directly (no numerator /
 * window-sum decomposition exists for |.|): CUDA-core kernels only, no ROI mode
 * (NCC_ERR_UNSUPPORTED), no flat-template flags. */
enum { NCC_SCORE_NCC = 0, NCC_SCORE_SSD = 1, NCC_SCORE_SAD = 2 };
enum { NCC_SUBPIX_GAUSS3 = 0, NCC_SUBPIX_PARABOLA3 = 1, NCC_SUBPIX_NONE = 2 };

/* ncc_problem.flags */
enum {
    NCC_F_WRITE_SURFACE = 1u,  /* TM: ncc_match writes the score surface (d_scores required) */
    NCC_F_GENERIC_KERNEL = 2u, /* force the run-time-evaluated (RE) generic kernels         */
    NCC_F_NO_JIT = 4u,         /* never compile at run time (NVRTC): AOT instance or generic */
    NCC_F_TIMING = 8u,         /* record per-stage CUDA-event timings (ncc_plan_timing)     */
    NCC_F_CUDA_CORES = 16u     /* TM: never use the tensor-core (tcgen05 3xTF32) numerator   */
};

/* Output flag bits (ncc_peak.flags, piv_vector.flags). */
enum {
    NCC_FLAG_FLAT_TEMPLATE = 1u, /* template (or PIV mask) has ~zero energy: no valid peak   */
    NCC_FLAG_EDGE_Y = 2u,        /* PIV peak on the search border in y: no sub-pixel fit     */
    NCC_FLAG_EDGE_X = 4u,        /* ... in x                                                 */
    NCC_FLAG_PARABOLA_Y = 8u,    /* PIV y fit used the parabolic fallback (a score <= 0)     */
    NCC_FLAG_PARABOLA_X = 16u,   /* ... x fit                                                */
    NCC_FLAG_INVALID = 32u       /* vector/peak is not meaningful (flat mask)                */
};

/* Problem statement (P:1290-1311 GPU-PF parameter analog). */
typedef struct {
    int32_t mode;    /* NCC_MODE_MATCH or NCC_MODE_PIV                                    */
    int32_t score;   /* NCC_SCORE_NCC or NCC_SCORE_SSD                                     */
    int32_t subpix;  /* PIV: NCC_SUBPIX_GAUSS3 (Gaussian, parabolic fallback) / PARABOLA3 / NONE */
    int32_t image_h; /* H: rows of every frame                                             */
    int32_t image_w; /* W: columns of every frame                                          */
    int64_t image_pitch; /* elements between rows, >= image_w                              */
    int32_t tmpl_h;  /* h: template (TM) or interrogation-window/mask (PIV) rows           */
    int32_t tmpl_w;  /* w: columns                                                          */
    int32_t search_y; /* PIV: radius m_y (offsets -m_y..+m_y); TM: must be 0 (all valid)   */
    int32_t search_x; /* PIV: radius m_x                                                     */
    int32_t step_y;  /* PIV: window step s_y (= (1-overlap)*window); TM: ignored           */
    int32_t step_x;  /* PIV: window step s_x                                               */
    int32_t batch;   /* TM: frames per call; PIV: frame pairs per call (per shard)        */
    int32_t shard_rank;  /* TM: band r = offset rows [r*U/n, (r+1)*U/n), n = shard_count;  */
                         /*     PIV: must be 0 (shard PIV by passing each rank its pairs) */
    int32_t shard_count; /* >= 1                                                            */
    uint32_t flags;  /* NCC_F_*                                                              */
    /* Multi-template / ROI matching (the paper's TM runtime operation: several templates per
     * frame, each searched within its region of interest -- Tab 5.1 caption P:190-191,
     * 5.1.3.4 P:91).  n_templates = 0 or 1 with roi_h = roi_w = 0: plain full/band search
     * (ncc_match).  n_templates >= 1 and roi_h, roi_w >= 1: ROI mode (ncc_match_rois), all
     * templates h x w, every (frame, template) searched over the offsets
     * [u0, u0+roi_h) x [v0, v0+roi_w) clipped to the valid range; shard_count must be 1. */
    int32_t n_templates;
    int32_t roi_h, roi_w;
} ncc_problem;

/* TM result per frame: argmax over the (band of) valid offsets, tie -> smallest u*V+v.
 * (u, v) are global (unsharded) offset coordinates.  flags: NCC_FLAG_FLAT_TEMPLATE |
 * NCC_FLAG_INVALID when the template is flat (then score = 0, u = u_begin, v = 0). */
typedef struct {
    float score;
    int32_t u, v;
    uint32_t flags;
} ncc_peak; /* 16 B */

/* PIV result per window, ordered [pair][k_y][k_x].  Window (k_y,k_x) has its mask origin
 * at (y, x) = (m_y + k_y*s_y, m_x + k_x*s_x); (dy, dx) is the displacement from frame A to
 * frame B: B(y+dy, x+dx) ~= A(y, x).  iy, ix: integer peak; dy, dx: sub-pixel. */
typedef struct {
    int32_t iy, ix;
    float dy, dx;
    float score;
    uint32_t flags;
} piv_vector; /* 24 B */

/* Read-only plan facts (ncc_plan_query). */
typedef struct {
    int32_t mode;
    int32_t U, V;              /* TM: offset grid; PIV: (2m_y+1), (2m_x+1)                  */
    int32_t u_begin, u_end;    /* TM: this shard's offset-row band                          */
    int32_t Ky, Kx;            /* PIV: window grid                                           */
    int32_t batch;
    int64_t outputs_per_call;  /* TM: band offsets x batch; PIV: Ky*Kx*batch vectors        */
    double flops_per_call;     /* algorithmic numerator FLOP per call (2hw per offset)      */
    int32_t specialized;       /* numerator tier: 1 = ahead-of-time specialised (SK) instance,
                                  2 = run-time specialised (NVRTC) kernel, 0 = generic run-time-
                                  evaluated (RE) kernel, 3 = tensor-core kernel (tcgen05 3xTF32;
                                  one kernel for every shape, h and w run-time evaluated)       */
    int32_t variant_id;        /* index into the variant table                              */
    int32_t regs_per_thread;   /* numerator kernel registers/thread                         */
    int32_t threads_per_block; /* numerator kernel block size                               */
    int32_t smem_per_block;    /* numerator kernel dynamic shared memory (bytes)            */
    int32_t grid_x, grid_y, grid_z; /* numerator launch grid (per sub-batch for PIV)        */
    int32_t launches_per_call; /* kernels this library launches per execute call          */
    int32_t split;             /* TM: split-K units per tile (accumulation order is fixed by it) */
    int32_t const_template;    /* TM: template read from the constant bank (1) or shared memory (0) */
    int32_t slabs;             /* TM: constant-bank template slabs (numerator launches)   */
    char variant_name[96];
} ncc_plan_info;

/* Per-stage device time of the most recent execute call (NCC_F_TIMING plans). */
typedef struct {
    float prep_ms;      /* template prep (TM; side stream, concurrent with stats) */
    float stats_ms;     /* call start -> window sums and template prep both done  */
    float numerator_ms; /* numerator + fused normalise/argmax (+ PIV sub-pixel)  */
    float finalize_ms;  /* peak finalisation (TM)                                */
    float total_ms;     /* whole call                                            */
    int32_t numerator_launches;
} ncc_timing;

/* Validate `p`, select the kernel variant for device `device`, allocate scratch.
 * Returns NCC_ERR_INVALID_ARGUMENT for: any size <= 0; h > H or w > W; pitch < W;
 * batch < 1; shard_count < 1 or shard_rank outside [0, shard_count) or a band with no
 * rows; PIV: search < 0, step <= 0, no window fits, shard_count != 1; TM: search != 0.
 * NCC_ERR_UNSUPPORTED when the problem needs more shared memory than the device has.
 * *out is NULL on failure. */
ncc_status ncc_plan_create(const ncc_problem* p, int device, ncc_plan* out);

/* TM on `batch` frames with one template.
 * d_images: batch frames (device); d_tmpl: h x w template, row pitch tmpl_pitch (elements).
 * d_scores: if NCC_F_WRITE_SURFACE, [batch][u_end-u_begin][V] fp32 surface (device), else
 *           ignored (may be NULL).  d_peaks: [batch] ncc_peak (device). */
ncc_status ncc_match(ncc_plan plan, const float* d_images, const float* d_tmpl,
                     int64_t tmpl_pitch, float* d_scores, ncc_peak* d_peaks, void* stream);

/* ROI mode (n_templates, roi_h, roi_w set): d_tmpls = n_templates templates, template t at
 * d_tmpls + t*tmpl_h*tmpl_pitch; d_rois = int32 [batch][n_templates][2] offset-space origins
 * (u0, v0) of the ROIs, each in [0, U) x [0, V) (device); d_scores (if NCC_F_WRITE_SURFACE)
 * [batch][n_templates][roi_h][roi_w] fp32; d_peaks [batch][n_templates], global (u, v),
 * argmax (NCC) / argmin (SSD) inside the clipped ROI, tie -> smallest u*V+v. */
ncc_status ncc_match_rois(ncc_plan plan, const float* d_images, const float* d_tmpls, int64_t tmpl_pitch,
                          const int32_t* d_rois, float* d_scores, ncc_peak* d_peaks, void* stream);

/* PIV on `batch` frame pairs: d_frames_a / d_frames_b (device), d_vectors [batch][Ky][Kx]. */
ncc_status piv_correlate(ncc_plan plan, const float* d_frames_a, const float* d_frames_b,
                         piv_vector* d_vectors, void* stream);

/* As piv_correlate, and also writes every window's score surface to d_scores
 * [batch][Ky][Kx][2m_y+1][2m_x+1] fp32 (device; NULL = do not write). */
ncc_status piv_correlate_ex(ncc_plan plan, const float* d_frames_a, const float* d_frames_b,
                            float* d_scores, piv_vector* d_vectors, void* stream);

/* Host-buffer variants (end-to-end path): copy inputs host->device into plan-owned
 * staging buffers on `stream`, run, and copy results device->host.  Pinned host memory
 * gives asynchronous copies (and, for ncc_match_host, copies captured into the launch
 * sequence: the template's copy overlaps the frames'); results are valid after the stream is
 * synchronised.  h_scores may be NULL (not copied back).  piv_correlate_host streams batches
 * larger than one sub-batch through two device slots (the copy of chunk c+1 overlaps the
 * correlation of chunk c on a plan-owned copy stream); the host buffers must stay valid until
 * the stream is synchronised. */
ncc_status ncc_match_host(ncc_plan plan, const float* h_images, const float* h_tmpl,
                          int64_t tmpl_pitch, float* h_scores, ncc_peak* h_peaks, void* stream);
ncc_status piv_correlate_host(ncc_plan plan, const float* h_frames_a, const float* h_frames_b,
                              piv_vector* h_vectors, void* stream);

/* Waits for the plan's outstanding work, frees everything.  NULL is allowed. */
ncc_status ncc_plan_destroy(ncc_plan plan);

const char* ncc_status_string(ncc_status s);
/* Message of the last CUDA error seen by this thread (empty string if none). */
const char* ncc_last_cuda_error(void);

/* Copies min(info_size, sizeof(ncc_plan_info)) bytes of plan facts into info. */
ncc_status ncc_plan_query(ncc_plan plan, void* info, size_t info_size);
/* Timings of the most recent execute call (requires NCC_F_TIMING; otherwise zeros). */
ncc_status ncc_plan_timing(ncc_plan plan, ncc_timing* out);

/* Run-time specialisation ahead of use (no device needed): selects the kernel variant for
 * *p exactly as ncc_plan_create would and, if that is a run-time specialised (NVRTC) kernel,
 * compiles it into the on-disk binary cache (NCC_CACHE_DIR, default ~/.cache/ncc_b200; the
 * paper's GPU-PF binary cache).  Writes the variant name (NUL-terminated) and
 * *compiled_now = 1 if NVRTC ran in this call (0: ahead-of-time instance or cache hit).
 * NCC_ERR_COMPILE if NVRTC is missing or fails (log in ncc_last_cuda_error); the plan would
 * then use the generic kernel. */
ncc_status ncc_specialize(const ncc_problem* p, char* variant_name, size_t name_size, int32_t* compiled_now);

/* Library build facts: 100 = sm_100a build. */
int32_t ncc_build_arch(void);

#ifdef __cplusplus
}
#endif
#endif /* NCC_B200_H */
