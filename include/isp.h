/*
 * isp.h -- C ABI of the B200 (sm_100a) border-handling stencil library libisp.so.
 *
 * Method: Qiao, Teich, Hannig, "An Efficient Approach for Image Border Handling on
 * GPUs via Iteration Space Partitioning", IPDPS 2021 (PAPER.md, cited "P:L<line>").
 * A local operator computes every output pixel of an sx x sy image
 * (iteration space x in [0,sx), y in [0,sy)) from an m x n window of input
 * pixels; reads that fall outside the image go through a global border pattern
 * (P:L34-37).  Iteration space partitioning (ISP, §III.C) splits the launch
 * into nine regions TL,T,TR,L,Body,R,BL,B,BR (Fig. 1); each region runs code with
 * only the bounds checks it needs (Body: none), selected per thread block
 * (Listing 3) or per warp (Listing 5).  The analytic model
 * (Eqs. 3-10) chooses ISP or the naive all-checks kernel ("isp+m").
 *
 * Conventions (all entry points):
 *  - Image buffers (img, out, dx, dy, ...) are DEVICE pointers owned by the caller,
 *    row-major with a row pitch given in ELEMENTS (pitch >= w).  A stencil cannot run
 *    in place: overlapping input/output ranges return ISP_EALIAS.
 *  - Masks / coefficient arrays are HOST pointers, read during the call and copied
 *    into the kernel's parameter block (no lifetime requirement after return).
 *  - Windows are odd, m x n with m along x (reading A8), 1 <= m, n <= 31; masks are
 *    row-major mask[j*m + i], multiplying the tap at offset (i - m/2, j - n/2)
 *    (correlation, reading A9).
 *  - Border modes (isp_border_t): Clamp, Mirror (symmetric, edge duplicated), Repeat
 *    (periodic), Constant (const_val for every out-of-bounds tap), defined for ANY
 *    window size, including windows larger than the image (readings A4-A7).
 *  - Every call is asynchronous and stream-ordered on `stream` (a cudaStream_t passed
 *    as void*; NULL = the legacy default stream); nothing synchronises except
 *    isp_shard_* barriers.  Calls never throw; they return an isp_status_t and leave a
 *    thread-local message in isp_last_error().  Launch failures return ISP_ECUDA.
 *  - Misaligned rows (base or pitch*sizeof(T) not a multiple of 16 B) are not an
 *    error: the kernels switch to scalar loads/stores; results are identical.
 *  - Results of ISP_BLOCK, ISP_WARP and ISP_NAIVE are bitwise identical (same
 *    arithmetic, only the index code differs).
 */
#ifndef ISP_H_
#define ISP_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum { ISP_CLAMP = 0, ISP_MIRROR = 1, ISP_REPEAT = 2, ISP_CONSTANT = 3 } isp_border_t;
typedef enum { ISP_U8 = 0, ISP_I16 = 1, ISP_I32 = 2, ISP_F32 = 3 } isp_dtype_t;
/* ISP_AUTO = "isp+m": the model of Eq. (10) picks ISP or NAIVE; its ISP is
 * ISP_TMA where eligible, else ISP_WARP.  ISP_BLOCK = Listing 3 and ISP_WARP = Listing 5
 * on the register-streaming kernels (per-read checks only where a region needs them);
 * ISP_TMA = Listing 3 on the staged kernels: for separable f32 masks (images and strips),
 * normalised separable u8 masks, Sobel, Laplace, Harris and the cfg3 pipeline the
 * warp-strip band kernels (per-warp shared-memory row rings filled by cp.async; a warp's
 * region from its strip / band: T / B rows mapped once per staged row, L / R edge lanes'
 * halo words, Body none; A34), otherwise the TMA-staged kernels (bulk async copies into
 * shared memory; checks only in the staging of border blocks, A21) -- each needs its
 * alignment (16 B for f32, 4-16 B per lane for u8 / i16) and a compiled window, else runs
 * as ISP_BLOCK; ISP_NAIVE = all four checks on every read (Eq. 3 baseline). */
/* Ablations: ISP_SPLIT = one kernel per region (the nine regions launched
 * separately over their block rectangles, instead of the paper's single fat kernel with
 * the Listing-3 switch; plans like ISP_BLOCK); ISP_TEX = texture hardware border
 * handling (every tap read through a texture object whose address mode implements
 * the pattern -- clamp, mirror, wrap, border colour; isp_filter_ex only, 2-D FMA order). */
typedef enum { ISP_AUTO = 0, ISP_BLOCK = 1, ISP_WARP = 2, ISP_NAIVE = 3, ISP_TMA = 4, ISP_SPLIT = 5,
               ISP_TEX = 6 } isp_variant_t;
typedef enum {
    ISP_OK = 0,
    ISP_EINVAL = 1,       /* bad size / pitch / window / mode / constant / divisor */
    ISP_EUNSUPPORTED = 2, /* dtype-filter combination not built */
    ISP_EALIAS = 3,       /* input and output ranges overlap */
    ISP_ECUDA = 4,        /* CUDA launch or runtime failure (see isp_last_error) */
    ISP_ENCCL = 5         /* NCCL failure in isp_shard_* */
} isp_status_t;

typedef void *isp_stream_t; /* cudaStream_t */

/* ---------------------------------------------------------------------------------
 * Generic f32 local operator (Mask with precomputed coefficients,
 * BoundaryCondition with pattern + constant, IterationSpace = whole image).
 *   out(x,y) = sum_{j,i} mask[j*mw+i] * in(B(x+i-mw/2), B(y+j-mh/2))   (f32 FMA,
 *   row-major tap order).  A rank-1 mask is detected and run as a separable pass;
 *   results then differ from the 2-D order only by f32 rounding.
 * isp_filter is the north-star convenience call: stream NULL, variant ISP_AUTO,
 * out has the same pitch as img.  isp_filter_naive forces ISP_NAIVE.
 * --------------------------------------------------------------------------------- */
isp_status_t isp_filter(const float *img, int w, int h, int pitch, const float *mask, int mw, int mh,
                        int border_mode, float const_val, float *out);
isp_status_t isp_filter_naive(const float *img, int w, int h, int pitch, const float *mask, int mw,
                              int mh, int border_mode, float const_val, float *out);
isp_status_t isp_filter_ex(const float *img, int w, int h, int pitch, const float *mask, int mw, int mh,
                           int border_mode, float const_val, float *out, int out_pitch,
                           isp_variant_t variant, isp_stream_t stream);

/* Separable f32 local operator: out = col (x) row applied as a row pass then a column
 * pass inside one kernel (no intermediate image), i.e. mask[j][i] = col[j]*row[i]. */
isp_status_t isp_filter_sep_f32(const float *img, int w, int h, int pitch, const float *row, int mw,
                                const float *col, int mh, int border_mode, float const_val, float *out,
                                int out_pitch, isp_variant_t variant, isp_stream_t stream);

/* u8 image, int32 mask: out = sat_u8( floor((2*acc + divisor) / (2*divisor)) ), i.e.
 * round-half-up of acc/divisor then saturate (reading A12).  Exact integer arithmetic:
 * bit-identical to the oracle.  divisor > 0; const_val in [0,255].  Binomial Gaussian:
 * mask b(x)b, divisor (sum b)^2 (a7); rank-1 integer masks run separably (exact). */
isp_status_t isp_filter_u8(const uint8_t *img, int w, int h, int pitch, const int32_t *mask, int mw,
                           int mh, int32_t divisor, int border_mode, int const_val, uint8_t *out,
                           int out_pitch, isp_variant_t variant, isp_stream_t stream);

/* Sobel (x-, y-derivative local operators + magnitude point operator), fused in
 * one pass over the u8 image: dx = img (*) [[-1,0,1],[-2,0,2],[-1,0,1]], dy with the
 * transpose (int16, exact), mag = min(255, round_half_up(sqrt(dx^2+dy^2))) (u8, exact
 * integer sqrt).  Any of dx, dy, mag may be NULL; all share out_pitch (elements). */
isp_status_t isp_sobel_u8(const uint8_t *img, int w, int h, int pitch, int border_mode, int const_val,
                          int16_t *dx, int16_t *dy, uint8_t *mag, int out_pitch, isp_variant_t variant,
                          isp_stream_t stream);

/* Laplace 5x5 (a8): mask of ones with centre -24, out = clamp(acc, 0, 255). */
isp_status_t isp_laplace5_u8(const uint8_t *img, int w, int h, int pitch, int border_mode, int const_val,
                             uint8_t *out, int out_pitch, isp_variant_t variant, isp_stream_t stream);

/* Harris response over Sobel derivatives (BASELINE.json configs[2]; not in the paper;
 * a10): 3x3 window, weights [1,2,1](x)[1,2,1]; Sxx, Syy, Sxy exact;
 * R25 = 25*(Sxx*Syy - Sxy^2) - (Sxx+Syy)^2 (k = 1/25, int64); out = R25 > thr ? 255 : 0.
 * dx, dy share `pitch`; border handling applies to the dx/dy images.
 * Domain (precondition): every dx, dy value and const_val lie in [-1020, 1020], the
 * range of 3x3 Sobel derivatives of u8 images.  Inside it the kernels evaluate R25
 * exactly (f32 window sums < 2^24, f64 response < 2^53)
 * and equal the int64 definition bit for bit at every thr.  const_val outside the
 * range returns ISP_EINVAL; device data outside it is not checked (results unspecified). */
isp_status_t isp_harris_u8(const int16_t *dx, const int16_t *dy, int w, int h, int pitch, int border_mode,
                           int const_val, int64_t thr, uint8_t *out, int out_pitch, isp_variant_t variant,
                           isp_stream_t stream);

/* BASELINE.json configs[2] fused into ONE launch (Sobel, Laplace from
 * P:L355, Harris a10): reads the u8 image once and writes mag, lap, harris (u8) and,
 * if non-NULL, dx and dy (int16).  Bit-identical to
 *   isp_sobel_u8(img, mode, const_val) -> dx, dy, mag;  isp_laplace5_u8(img, mode, const_val);
 *   isp_harris_u8(dx, dy, mode, harris_const, thr)
 * i.e. Harris' border handling applies to the dx/dy IMAGES (remapped coordinates).
 * All outputs share out_pitch (elements); img is caller-owned device memory, pitch in
 * bytes = elements.  ISP_NAIVE stages every tile through the checked gather; any other
 * variant runs Body tiles unchecked.  EINVAL: sizes/pitches, mode, NULL mag/lap/harris,
 * const_val not in [0,255], harris_const not in [-1020,1020] (the Sobel range; keeps the
 * int32 window sums exact).  EALIAS: an output overlaps img.  Stream-ordered. */
isp_status_t isp_pipeline_cfg3_u8(const uint8_t *img, int w, int h, int pitch, int border_mode, int const_val,
                                  int harris_const, int64_t thr, int16_t *dx, int16_t *dy, uint8_t *mag,
                                  uint8_t *lap, uint8_t *harris, int out_pitch, isp_variant_t variant,
                                  isp_stream_t stream);

/* Bilateral filter (a11), f32, window win x win (odd, <= 31):
 *   out(p) = sum_q s(q-p) r(I_q-I_p) I_q / sum_q s(q-p) r(I_q-I_p),
 *   s = exp(-(dx^2+dy^2)/(2 sigma_d^2)), r(d) = exp(-d^2/(2 sigma_r^2)).
 * Tolerance vs the double oracle: max-abs 1e-4 on [0,1] data. */
isp_status_t isp_bilateral_f32(const float *img, int w, int h, int pitch, int win, float sigma_d,
                               float sigma_r, int border_mode, float const_val, float *out, int out_pitch,
                               isp_variant_t variant, isp_stream_t stream);

/* Atrous pass of the Night filter (a12, coefficients ours, reading A26):
 * out = sum_{i,j in {-1,0,1}} h_i h_j in(B(x+d*i), B(y+d*j)), h = [1,2,1]/4, dilation
 * d in {1,2,4,8}.  tonemap != 0 fuses the Night tone map t(v) = v/(1+v) (point op). */
isp_status_t isp_atrous_f32(const float *img, int w, int h, int pitch, int dilation, int border_mode,
                            float const_val, int tonemap, float *out, int out_pitch, isp_variant_t variant,
                            isp_stream_t stream);

/* Night filter: Atrous d = 1, 2, 4, 8 then tone mapping; tmp0/tmp1 are
 * caller-owned f32 scratch images of the same geometry (pitch = out_pitch). */
isp_status_t isp_night_f32(const float *img, int w, int h, int pitch, int border_mode, float const_val,
                           float *tmp0, float *tmp1, float *out, int out_pitch, isp_variant_t variant,
                           isp_stream_t stream);

/* ---------------------------------------------------------------------------------
 * Planner introspection (pure host; no GPU needed when occupancies are supplied).
 * Eq. (2) bounds (reading A2), Eq. (7)/(8) counts (A17), warp bounds (Listing 5, A22),
 * Eqs. (3)-(6), (9), (10) model (A13-A15, A18-A20).
 * --------------------------------------------------------------------------------- */
typedef struct {
    int bh_l, bh_r, bh_t, bh_b;  /* Eq. (2) block bounds */
    int nx, ny;                  /* Eq. (7) blocks per dimension */
    int w_l, w_r;                /* warp-column bounds (global warp columns) */
    int degenerate;              /* BH_L > BH_R or BH_T > BH_B (A3): NAIVE is used */
    long long n_block[9];        /* Eq. (8), order TL,TR,T,BL,BR,B,R,L,Body (Eq. 4) */
    double n_naive, n_isp;       /* Eqs. (3), (4) */
    double r_reduced, o_naive, o_isp, g; /* Eqs. (9), (10) */
    isp_variant_t choice;        /* ISP_WARP/ISP_BLOCK if G > 1, else ISP_NAIVE */
    int tile_w, tile_h, warp_w;  /* tile (block) and warp widths in pixels */
} isp_plan_info;

/* Model inputs.  n_check / n_kernel: instructions per border check / per tap of the
 * kernel; ipc_switch: instructions per Listing-3 compare (A18); o_*: occupancy
 * in [0,1] -- pass <= 0 to query the CUDA occupancy API for the kernels this library
 * would launch (needs a GPU).  form: 0 = per-thread switch (A14 "T"), 1 = as printed,
 * 2 = staged (checks per staged element, A21), 3 = band (checks per staged row, A34). */
typedef struct {
    double n_check, n_kernel, ipc_switch, o_naive, o_isp;
    int form;
} isp_model_params;

/* filter_id: 0 generic f32, 1 separable f32, 2 u8, 3 sobel, 4 laplace5, 5 harris,
 * 6 bilateral, 7 atrous.  tile_w/tile_h <= 0 selects the library's launch tile. */
isp_status_t isp_plan(int w, int h, int mw, int mh, int tile_w, int tile_h, int warp_w, int border_mode,
                      int filter_id, const isp_model_params *params, isp_plan_info *out);
/* Sparse masks (the paper's future work P:L394; reading A31).  reach =
 * {left, right, top, bottom}: how far the NON-ZERO taps of an odd mw x mh mask reach
 * beyond its centre anchor (clamped at 0).  isp_filter_ex / isp_filter_u8 crop masks with
 * all-zero edge rows / columns to this footprint (zero taps add exactly 0 on finite
 * images, so results are unchanged) and take the ISP bounds from it.  dtype: ISP_F32
 * (float mask) or ISP_I32 (int32 mask).  Pure host. */
isp_status_t isp_mask_reach(const void *mask, int dtype, int mw, int mh, int reach[4]);
/* Eq. (2) with per-side reaches (reading A31): BH_L = ceil(L/tx), BH_R = floor((w-R)/tx),
 * BH_T = ceil(T/ty), BH_B = floor((h-B)/ty), warp bounds likewise, Eq. (8) block counts.
 * tile_w = tx (pixels), tile_h = ty (rows), warp_w = warp width in pixels (<= 0: tx).
 * Pure host; model fields are not filled (choice = ISP_BLOCK, or ISP_NAIVE if degenerate). */
isp_status_t isp_plan_reach(int w, int h, const int reach[4], int tile_w, int tile_h, int warp_w,
                            isp_plan_info *out);
/* Default model constants for a filter/mode (calibration). */
isp_status_t isp_model_defaults(int filter_id, int border_mode, int mw, int mh, isp_model_params *out);

/* ---------------------------------------------------------------------------------
 * Multi-GPU row strips (not in the paper).  One process per GPU.
 * Rank r owns output rows [y0_r, y0_r + strip_h_r) with y0_r = r*ceil(H/P) (last rank
 * shorter).  The caller's strip buffer holds (strip_h + 2*halo) rows of `pitch`
 * elements: rows [0, halo) receive the upper neighbour's rows, rows
 * [halo, halo+strip_h) are the rank's own input rows, rows [halo+strip_h, ...) the
 * lower neighbour's.  isp_shard_filter_f32 exchanges the halos with NCCL send/recv
 * (ring wrap for Repeat) on `comm_stream`, filters the interior rows on `stream`
 * meanwhile, then the 2*halo rows next to the strip edges; only rank 0 has the image
 * T border and rank P-1 the B border.  Output: strip_h rows of out_pitch.
 * --------------------------------------------------------------------------------- */
typedef struct isp_shard_ctx isp_shard_ctx;

/* Pure-host schedule of one rank (no GPU / NCCL needed; tests check it on CPU).
 * ops: NCCL point-to-point calls in issue order; kind 0 = send, 1 = recv; `row` is the
 * first strip-buffer row, `nrows` rows of `pitch` elements.  launch: filter launches
 * over global output rows [oy0, oy0+nrows); reads limited to rows < ylim; t_real /
 * b_real: the launch's top / bottom edge is a real image border; after_halo: the
 * launch waits for the exchange. */
typedef struct { int kind, peer, row, nrows; } isp_shard_op;
typedef struct { int oy0, nrows, ylim, t_real, b_real, after_halo; } isp_shard_launch;
typedef struct {
    int y0, strip_h, prev, next, n_ops, n_launch;
    isp_shard_op ops[4];
    isp_shard_launch launch[3];
} isp_shard_sched;
isp_status_t isp_shard_schedule(int H, int rank, int nranks, int halo, int hy, int border_mode,
                                isp_shard_sched *out);
isp_status_t isp_shard_unique_id(unsigned char id[128]);
isp_status_t isp_shard_init(isp_shard_ctx **ctx, const unsigned char id[128], int rank, int nranks,
                            int device);
/* Row range owned by `rank` for an image of height H split over nranks ranks. */
isp_status_t isp_shard_rows(int H, int rank, int nranks, int *y0, int *strip_h);
isp_status_t isp_shard_filter_f32(isp_shard_ctx *ctx, float *strip, int w, int H, int pitch, int halo,
                                  const float *mask, int mw, int mh, int border_mode, float const_val,
                                  float *out, int out_pitch, isp_variant_t variant, isp_stream_t stream,
                                  isp_stream_t comm_stream);
isp_status_t isp_shard_filter_u8(isp_shard_ctx *ctx, uint8_t *strip, int w, int H, int pitch, int halo,
                                 const int32_t *mask, int mw, int mh, int32_t divisor, int border_mode,
                                 int const_val, uint8_t *out, int out_pitch, isp_variant_t variant,
                                 isp_stream_t stream, isp_stream_t comm_stream);
/* The launch part of isp_shard_filter_f32 for rank `rank` of `nranks`, without any
 * communication: the caller has already filled the strip's halo rows (e.g. its own
 * exchange, or a single-GPU emulation of the strips in tests). */
isp_status_t isp_shard_filter_local_f32(float *strip, int w, int H, int pitch, int halo, int rank, int nranks,
                                        const float *mask, int mw, int mh, int border_mode, float const_val,
                                        float *out, int out_pitch, isp_variant_t variant, isp_stream_t stream);
/* Only the halo exchange of isp_shard_filter_* (the schedule's NCCL send/recv, rows of
 * `pitch` elements of `elem_size` bytes) on comm_stream -- for timing the exchange alone
 * and for callers that run their own launches.  Stream-ordered; no filtering. */
isp_status_t isp_shard_exchange(isp_shard_ctx *ctx, void *strip, int elem_size, int H, int pitch, int halo, int hy,
                                int border_mode, isp_stream_t comm_stream);
/* Peer-direct strips: each rank's `strip` holds ONLY its own strip_h rows
 * (pitch elements each, no halo rows); the hy rows above / below are read straight from the
 * neighbour ranks' strips in peer memory (CUDA IPC mappings over NVLink), so one launch
 * covers the strip and no halo exchange runs.  Only rank 0 / P-1 own the image T / B
 * borders (Repeat: the ring neighbours supply the wrapped rows).
 *   isp_shard_peer_open: collective over the ctx's ranks (NCCL all-gather of the IPC
 *     handles of every rank's strip allocation); ring != 0 also maps the wrap neighbours
 *     (needed for Repeat).  The strip must stay allocated until isp_shard_peer_close.
 *   Ordering contract: every rank's strip must hold its data before any rank's filter
 *     call starts (e.g. a process-group barrier after writing them) and must not be
 *     rewritten until the neighbours' calls have finished.
 *   isp_shard_filter_peer_local_*: the same launch with explicit neighbour pointers
 *     (prev = rank r-1's strip, next = rank r+1's, ring neighbours for Repeat at the ends;
 *     any pointers the device can read -- single-GPU emulation in tests).
 * f32 and u8 filters (isp_filter_ex / isp_filter_u8 semantics, all variants except TEX). */
typedef struct isp_shard_peer isp_shard_peer;
isp_status_t isp_shard_peer_open(isp_shard_ctx *ctx, void *strip, int ring, isp_shard_peer **out);
/* The two halves of isp_shard_peer_open for callers that exchange the 72-byte handles
 * themselves (e.g. over a gloo process group): the handle of this rank's strip, and the
 * attach of the neighbours given every rank's handle (nranks x 72 bytes, rank order). */
isp_status_t isp_shard_peer_handle(void *strip, unsigned char out[72]);
isp_status_t isp_shard_peer_attach(int rank, int nranks, int device, void *strip, const unsigned char *handles,
                                   int ring, isp_shard_peer **out);
isp_status_t isp_shard_peer_filter_f32(isp_shard_peer *peer, int w, int H, int pitch, const float *mask, int mw,
                                       int mh, int border_mode, float const_val, float *out, int out_pitch,
                                       isp_variant_t variant, isp_stream_t stream);
isp_status_t isp_shard_peer_close(isp_shard_peer *peer);
isp_status_t isp_shard_filter_peer_local_f32(const float *own, const float *prev, const float *next, int w, int H,
                                             int pitch, int rank, int nranks, const float *mask, int mw, int mh,
                                             int border_mode, float const_val, float *out, int out_pitch,
                                             isp_variant_t variant, isp_stream_t stream);
isp_status_t isp_shard_filter_peer_local_u8(const uint8_t *own, const uint8_t *prev, const uint8_t *next, int w,
                                            int H, int pitch, int rank, int nranks, const int32_t *mask, int mw,
                                            int mh, int32_t divisor, int border_mode, int const_val, uint8_t *out,
                                            int out_pitch, isp_variant_t variant, isp_stream_t stream);
/* u8 counterpart of isp_shard_filter_local_f32 (the launch part of isp_shard_filter_u8). */
isp_status_t isp_shard_filter_local_u8(uint8_t *strip, int w, int H, int pitch, int halo, int rank, int nranks,
                                       const int32_t *mask, int mw, int mh, int32_t divisor, int border_mode,
                                       int const_val, uint8_t *out, int out_pitch, isp_variant_t variant,
                                       isp_stream_t stream);
isp_status_t isp_shard_destroy(isp_shard_ctx *ctx);

/* Tuning: force the launch shape (warps per block along x, tile height in rows);
 * 0 restores the planner default.  Process-global, not thread-safe. */
isp_status_t isp_set_launch_override(int warps_x, int tile_h);

/* Last launch's resolved plan on this thread (which variant/tile AUTO picked). */
isp_status_t isp_last_plan(isp_plan_info *out);
/* The last min(n, 16) resolved launch plans of this thread, oldest first (multi-launch
 * calls: isp_night_f32, isp_shard_*); returns how many were written.
 * isp_clear_plans forgets them (tests). */
int isp_recent_plans(isp_plan_info *out, int n);
void isp_clear_plans(void);
const char *isp_status_string(isp_status_t s);
const char *isp_last_error(void); /* thread-local */
int isp_version(void);

#ifdef __cplusplus
}
#endif
#endif /* ISP_H_ */
