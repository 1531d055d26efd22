/*
 * isp_oracle.c -- plain, slow, obviously-correct CPU oracle for the ISP hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library.  It shares no
 * code, header, table or helper with the CUDA path (paper_conf_ipps_qiaoth21_b200/)
 * and never calls it.
 *
 * Source: Qiao, Teich, Hannig, "An Efficient Approach for Image Border Handling on
 * GPUs via Iteration Space Partitioning", IPDPS 2021 (/root/reference/PAPER.md,
 * cited "P:L<line>").  ISP is an exact transformation: it must
 * produce the naive result.  So this oracle is the PLAIN DEFINITION with no
 * partitioning at all:
 *
 *     out(x,y) = F( { in(B_x(x+i-hx), B_y(y+j-hy)) : 0<=i<m, 0<=j<n } )
 *
 * for every (x,y) in [0,sx) x [0,sy) (iteration space), with the border
 * pattern B applied on EVERY read.  Readings of garbled/silent points
 * are numbered A<k> as in SURVEY.md §8(c) and DESIGN.md "Readings".
 *
 * Floating point: accumulation in double, row-major tap order.  Integer paths use
 * exact (64-bit) integer arithmetic.  Every function computes output rows
 * [y0, y1) only, written densely to out[(y-y0)*w + x], so large images can be
 * validated on sampled rows.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>

#define ORC_CLAMP 0
#define ORC_MIRROR 1
#define ORC_REPEAT 2
#define ORC_CONSTANT 3

/* ------------------------------------------------------------------------- */
/* Border index map B_mode(i, N)  (§III.A, Fig. 2; Listing 1 missing) */
/* Returns the in-range index, or -1 for "use the constant" (Constant pattern). */
/* ------------------------------------------------------------------------- */
long orc_border_index(int mode, long i, long N)
{
    if (i >= 0 && i < N) return i;
    switch (mode) {
    case ORC_CLAMP:      /* "returns the nearest valid pixel within bounds"; A6 */
        return i < 0 ? 0 : N - 1;
    case ORC_MIRROR: {   /* "mirrored pixels at the border"; A4: symmetric,
                            edge duplicated, period 2N for any overshoot */
        long p = 2 * N;
        long r = i % p;
        if (r < 0) r += p;
        return r < N ? r : p - 1 - r;
    }
    case ORC_REPEAT: {   /* "tile the image with itself ... periodically"; A5 */
        long r = i % N;
        if (r < 0) r += N;
        return r;
    }
    case ORC_CONSTANT:   /* "user-defined value for all out of bounds pixels"; A7 */
        return -1;
    default:
        return -2;
    }
}

/* Read one pixel of a float image through the border map (Constant: a tap is C
 * iff x or y is out of bounds, A7). */
static double rd_f32(const float *img, long w, long h, long pitch, int mode, double C, long x, long y)
{
    long bx = orc_border_index(mode, x, w), by = orc_border_index(mode, y, h);
    if (bx < 0 || by < 0) return C;
    return (double)img[by * pitch + bx];
}

static long rd_u8(const uint8_t *img, long w, long h, long pitch, int mode, long C, long x, long y)
{
    long bx = orc_border_index(mode, x, w), by = orc_border_index(mode, y, h);
    if (bx < 0 || by < 0) return C;
    return (long)img[by * pitch + bx];
}

static long rd_i16(const int16_t *img, long w, long h, long pitch, int mode, long C, long x, long y)
{
    long bx = orc_border_index(mode, x, w), by = orc_border_index(mode, y, h);
    if (bx < 0 || by < 0) return C;
    return (long)img[by * pitch + bx];
}

static int bad_args(long w, long h, long pitch, int mw, int mh, int mode)
{
    return w < 1 || h < 1 || pitch < w || mw < 1 || mh < 1 || (mw % 2) == 0 || (mh % 2) == 0
        || mode < 0 || mode > 3;
}

/* ------------------------------------------------------------------------- */
/* Generic local operator with a float mask (correlation, A9), double accumulation. */
/* mask[j*mw + i] multiplies the tap at offset (i-hx, j-hy) (A8).                 */
/* scale_out (optional) receives sum_taps |mask*in| per pixel, the denominator of */
/* the f32 relative tolerance (A28).                                              */
/* ------------------------------------------------------------------------- */
int orc_filter_f64(const float *img, int w, int h, long pitch, const double *mask, int mw, int mh,
                   int mode, double C, int y0, int y1, double *out, double *scale_out)
{
    if (bad_args(w, h, pitch, mw, mh, mode) || y0 < 0 || y1 > h || y0 > y1) return 1;
    int hx = mw / 2, hy = mh / 2;
    for (long y = y0; y < y1; ++y)
        for (long x = 0; x < w; ++x) {
            double acc = 0.0, sc = 0.0;
            for (int j = 0; j < mh; ++j)
                for (int i = 0; i < mw; ++i) {
                    double v = rd_f32(img, w, h, pitch, mode, C, x + i - hx, y + j - hy);
                    double t = mask[j * mw + i] * v;
                    acc += t;
                    sc += fabs(t);
                }
            out[(y - y0) * w + x] = acc;
            if (scale_out) scale_out[(y - y0) * w + x] = sc;
        }
    return 0;
}

/* ------------------------------------------------------------------------- */
/* u8 image, integer mask: out = sat_u8( round_half_up(acc / divisor) )          */
/* round_half_up(a/d) = floor((2a + d) / (2d))  (A12), exact 64-bit integers.     */
/* ------------------------------------------------------------------------- */
static long floor_div(long a, long b) /* b > 0 */
{
    long q = a / b, r = a % b;
    return (r != 0 && r < 0) ? q - 1 : q;
}

int orc_filter_u8(const uint8_t *img, int w, int h, long pitch, const int32_t *mask, int mw, int mh,
                  int32_t divisor, int mode, int C, int y0, int y1, uint8_t *out)
{
    if (bad_args(w, h, pitch, mw, mh, mode) || divisor <= 0 || C < 0 || C > 255 || y0 < 0 || y1 > h
        || y0 > y1)
        return 1;
    int hx = mw / 2, hy = mh / 2;
    for (long y = y0; y < y1; ++y)
        for (long x = 0; x < w; ++x) {
            long acc = 0;
            for (int j = 0; j < mh; ++j)
                for (int i = 0; i < mw; ++i)
                    acc += (long)mask[j * mw + i] * rd_u8(img, w, h, pitch, mode, C, x + i - hx, y + j - hy);
            long q = floor_div(2 * acc + divisor, 2L * divisor);
            if (q < 0) q = 0;
            if (q > 255) q = 255;
            out[(y - y0) * w + x] = (uint8_t)q;
        }
    return 0;
}

/* u8 image, integer mask, raw integer sums (Sobel derivatives; a9). */
int orc_correlate_u8_i32(const uint8_t *img, int w, int h, long pitch, const int32_t *mask, int mw,
                         int mh, int mode, int C, int y0, int y1, int32_t *out)
{
    if (bad_args(w, h, pitch, mw, mh, mode) || C < 0 || C > 255 || y0 < 0 || y1 > h || y0 > y1) return 1;
    int hx = mw / 2, hy = mh / 2;
    for (long y = y0; y < y1; ++y)
        for (long x = 0; x < w; ++x) {
            long acc = 0;
            for (int j = 0; j < mh; ++j)
                for (int i = 0; i < mw; ++i)
                    acc += (long)mask[j * mw + i] * rd_u8(img, w, h, pitch, mode, C, x + i - hx, y + j - hy);
            out[(y - y0) * w + x] = (int32_t)acc;
        }
    return 0;
}

/* ------------------------------------------------------------------------- */
/* Sobel magnitude (point operator, 3rd Sobel kernel; a9):               */
/*   mag = min(255, round_half_up(sqrt(dx^2 + dy^2)))                            */
/* with an exact integer square root by bisection (no floating point).           */
/* ------------------------------------------------------------------------- */
static long isqrt_floor(long n)
{
    long lo = 0, hi = 1;
    while (hi * hi <= n) hi *= 2;
    while (hi - lo > 1) { /* invariant lo^2 <= n < hi^2 */
        long mid = lo + (hi - lo) / 2;
        if (mid * mid <= n) lo = mid; else hi = mid;
    }
    return lo;
}

int orc_sobel_mag(const int32_t *dx, const int32_t *dy, long n, uint8_t *out)
{
    for (long k = 0; k < n; ++k) {
        long s = (long)dx[k] * dx[k] + (long)dy[k] * dy[k];
        long r = isqrt_floor(s);
        /* round half up: sqrt(s) >= r + 1/2  <=>  s >= r^2 + r + 1/4  <=>  s > r^2 + r */
        if (s > r * r + r) r += 1;
        out[k] = (uint8_t)(r > 255 ? 255 : r);
    }
    return 0;
}

/* ------------------------------------------------------------------------- */
/* Harris corner response (BASELINE.json configs[2]; NOT in the paper; a10, A27). */
/* Local operator over (dx, dy) int16 images, window 3x3, weights w = b3 (x) b3: */
/*   Sxx = sum w dx^2, Syy = sum w dy^2, Sxy = sum w dx dy                        */
/*   R25 = 25 (Sxx Syy - Sxy^2) - (Sxx + Syy)^2      (= 25 * R with k = 1/25)     */
/*   out = R25 > thr ? 255 : 0                                                    */
/* Each read of dx/dy goes through the border map of the dx/dy images.           */
/* ------------------------------------------------------------------------- */
int orc_harris(const int16_t *dx, const int16_t *dy, int w, int h, long pitch, int mode, int C,
               int64_t thr, int y0, int y1, uint8_t *out)
{
    static const long b3[3] = {1, 2, 1};
    if (bad_args(w, h, pitch, 3, 3, mode) || y0 < 0 || y1 > h || y0 > y1) return 1;
    for (long y = y0; y < y1; ++y)
        for (long x = 0; x < w; ++x) {
            int64_t sxx = 0, syy = 0, sxy = 0;
            for (int j = 0; j < 3; ++j)
                for (int i = 0; i < 3; ++i) {
                    int64_t wt = b3[j] * b3[i];
                    int64_t gx = rd_i16(dx, w, h, pitch, mode, C, x + i - 1, y + j - 1);
                    int64_t gy = rd_i16(dy, w, h, pitch, mode, C, x + i - 1, y + j - 1);
                    sxx += wt * gx * gx;
                    syy += wt * gy * gy;
                    sxy += wt * gx * gy;
                }
            int64_t r25 = 25 * (sxx * syy - sxy * sxy) - (sxx + syy) * (sxx + syy);
            out[(y - y0) * w + x] = r25 > thr ? 255 : 0;
        }
    return 0;
}

/* ------------------------------------------------------------------------- */
/* Bilateral filter ("two convolutions together ... spatial closeness   */
/* ... intensity similarity"; a11):                                              */
/*   out(p) = sum_q s(q-p) r(I_q - I_p) I_q / sum_q s(q-p) r(I_q - I_p)         */
/*   s(dx,dy) = exp(-(dx^2+dy^2) / (2 sigma_d^2)),  r(d) = exp(-d^2/(2 sigma_r^2)) */
/* Out-of-bounds taps read through the border map; Constant taps are C (A7).     */
/* The centre pixel p itself is always in bounds.                                */
/* ------------------------------------------------------------------------- */
int orc_bilateral(const float *img, int w, int h, long pitch, int win, double sigma_d, double sigma_r,
                  int mode, double C, int y0, int y1, double *out)
{
    if (bad_args(w, h, pitch, win, win, mode) || !(sigma_d > 0) || !(sigma_r > 0) || y0 < 0 || y1 > h
        || y0 > y1)
        return 1;
    int hw = win / 2;
    for (long y = y0; y < y1; ++y)
        for (long x = 0; x < w; ++x) {
            double ip = (double)img[y * pitch + x];
            double num = 0.0, den = 0.0;
            for (int j = -hw; j <= hw; ++j)
                for (int i = -hw; i <= hw; ++i) {
                    double iq = rd_f32(img, w, h, pitch, mode, C, x + i, y + j);
                    double s = exp(-((double)(i * i + j * j)) / (2.0 * sigma_d * sigma_d));
                    double d = iq - ip;
                    double r = exp(-(d * d) / (2.0 * sigma_r * sigma_r));
                    num += s * r * iq;
                    den += s * r;
                }
            out[(y - y0) * w + x] = num / den;
        }
    return 0;
}

/* ------------------------------------------------------------------------- */
/* Atrous ("with holes") pass of the Night filter (ref 28; a12, A26):   */
/*   out = sum_{i,j in {-1,0,1}} h_i h_j in(B(x + d i), B(y + d j)),             */
/*   h = [1, 2, 1] / 4, dilation d = 2^(k-1) (windows 3, 5, 9, 17 for k=1..4).   */
/* ------------------------------------------------------------------------- */
int orc_atrous(const float *img, int w, int h, long pitch, int d, int mode, double C, int y0, int y1,
               double *out)
{
    static const double hk[3] = {0.25, 0.5, 0.25};
    if (bad_args(w, h, pitch, 1, 1, mode) || d < 1 || y0 < 0 || y1 > h || y0 > y1) return 1;
    for (long y = y0; y < y1; ++y)
        for (long x = 0; x < w; ++x) {
            double acc = 0.0;
            for (int j = -1; j <= 1; ++j)
                for (int i = -1; i <= 1; ++i)
                    acc += hk[j + 1] * hk[i + 1] * rd_f32(img, w, h, pitch, mode, C, x + d * i, y + d * j);
            out[(y - y0) * w + x] = acc;
        }
    return 0;
}

/* Night tone-mapping point operator ("actual tone mapping"; formula ours:
 * A26, parity unpinned against the paper):  t(v) = v / (1 + v). */
int orc_tonemap(const double *in, long n, double *out)
{
    for (long k = 0; k < n; ++k) out[k] = in[k] / (1.0 + in[k]);
    return 0;
}

int orc_version(void) { return 1; }
