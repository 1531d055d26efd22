// fused_cfg3.cu -- BASELINE.json configs[2] as ONE kernel: Sobel
// (dx, dy, magnitude), Laplace 5x5 and Harris over (dx, dy) from a single read of the u8
// image.  Output bits equal the three-launch pipeline isp_sobel_u8 -> isp_laplace5_u8 ->
// isp_harris_u8 (and the oracle composition oracle.sobel / laplace5_u8 / harris):
//
//   * Laplace and Sobel read img(B(x+i), B(y+j)): the staged input tile holds
//     exactly those values (C for Constant).
//   * Harris reads dx/dy at (B(x+i), B(y+j)) of the dx/dy IMAGES.  Inside the image that
//     is the Sobel value at an in-image pixel, recomputed from the staged tile.  Outside
//     it ("remapped coordinates") it is the Sobel value at the remapped pixel B(c) -- a
//     different pixel than a shifted window would give (Repeat: the opposite edge) -- so
//     those ext positions are evaluated by a checked global gather; Constant gives the
//     Harris constant instead.  Only border tiles have such positions.
//
// ISP at tile granularity (staged family, a6): Body tiles (whole staged window inside
// the image) stage with unchecked 16-byte loads; border tiles stage with a per-byte
// border-mapped gather (the region's checks).  ISP_NAIVE gathers on every tile.
//
// CTA = 128 threads = one output column each, TH rows; the thread walks down its column
// with register rings (no shared-memory re-reads across rows).
#include <cuda_runtime.h>
#include <stdint.h>

#include <cstring>

#include "../../include/isp.h"
#include "internal.h"

namespace {

constexpr int TW = 128;                // output columns per CTA (= threads)
constexpr int TH = 32;                 // output rows per CTA
constexpr int XO = 16;                 // staged input starts at x0 - XO (16-byte aligned)
constexpr int SW = TW + 2 * XO;        // staged row width (bytes)
constexpr int SH = TH + 4;             // staged rows: y0-2 .. y0+TH+1
constexpr int EW = TW + 2, EH = TH + 2;  // dx/dy ext: x0-1 .. x0+TW, y0-1 .. y0+TH

__device__ __forceinline__ int bmap(int mode, int i, int n)
{
    if (i >= 0 && i < n) return i;
    switch (mode) {
    case ISP_CLAMP: return i < 0 ? 0 : n - 1;
    case ISP_MIRROR: {
        const int p = 2 * n;
        int r = i % p;
        if (r < 0) r += p;
        return r < n ? r : p - 1 - r;
    }
    case ISP_REPEAT: {
        int r = i % n;
        if (r < 0) r += n;
        return r;
    }
    default: return -1;  // Constant
    }
}

__device__ __forceinline__ int rd_img(const uint8_t *img, int w, int h, int pitch, int mode, int cval, int x, int y)
{
    const int bx = bmap(mode, x, w), by = bmap(mode, y, h);
    if (bx < 0 || by < 0) return cval;
    return img[(size_t)by * pitch + bx];
}

// Exact round-half-up sqrt, clamped to 255 (a9): integer correction of the f32 estimate.
__device__ __forceinline__ int mag_u8(int n)
{
    if (n >= 65025 + 255) return 255;  // sqrt(n) >= 255.5 <=> n > 255^2 + 255
    int r = (int)sqrtf((float)n);
    while (r * r > n) --r;
    while ((r + 1) * (r + 1) <= n) ++r;
    return n > r * r + r ? r + 1 : r;
}

struct Params {
    const uint8_t *img;
    int w, h, pitch, mode, cval, hcval, out_pitch, naive, vec;
    long long thr;
    int16_t *dx, *dy;
    uint8_t *mag, *lap, *har;
};

__global__ void __launch_bounds__(TW) k_fused_cfg3(const Params p)
{
    __shared__ __align__(16) uint8_t s_in[SH][SW];
    __shared__ int16_t s_dx[EH][EW + 2], s_dy[EH][EW + 2];

    const int tid = threadIdx.x;
    const int x0 = blockIdx.x * TW, y0 = blockIdx.y * TH;
    const int w = p.w, h = p.h;

    // ---- stage img(B(x), B(y)) for x in [x0-2, x0+TW+2), y in [y0-2, y0+TH+2) ----------
    const bool body = !p.naive && p.vec && x0 - XO >= 0 && x0 + TW + XO <= w && y0 - 2 >= 0 && y0 + TH + 2 <= h;
    if (body) {
        constexpr int VPR = SW / 16;
        for (int k = tid; k < SH * VPR; k += TW) {
            const int r = k / VPR, c = k % VPR;
            const uint4 v = __ldg(reinterpret_cast<const uint4 *>(p.img + (size_t)(y0 - 2 + r) * p.pitch + x0 - XO) + c);
            *reinterpret_cast<uint4 *>(&s_in[r][c * 16]) = v;
        }
    } else {
        constexpr int GW = TW + 4;
        for (int k = tid; k < SH * GW; k += TW) {
            const int r = k / GW, c = k % GW;
            s_in[r][XO - 2 + c] = (uint8_t)rd_img(p.img, w, h, p.pitch, p.mode, p.cval, x0 - 2 + c, y0 - 2 + r);
        }
    }
    __syncthreads();

    // ---- dx, dy on the ext grid (column walk, 3-row ring) --------------------------------
    for (int c = tid; c < EW; c += TW) {
        const int sc = XO - 1 + c;  // s_in column of gx
        int d0 = 0, d1 = 0, s0 = 0, s1 = 0;
#pragma unroll
        for (int r = 0; r < EH + 2; ++r) {  // s_in rows 0 .. EH+1 (= y0-2 .. y0+TH+1)
            const int a = s_in[r][sc - 1], b = s_in[r][sc], cc = s_in[r][sc + 1];
            const int d2 = cc - a, s2 = a + 2 * b + cc;
            if (r >= 2) {
                s_dx[r - 2][c] = (int16_t)(d0 + 2 * d1 + d2);
                s_dy[r - 2][c] = (int16_t)(s2 - s0);
            }
            d0 = d1; d1 = d2; s0 = s1; s1 = s2;
        }
    }
    // border tiles: ext positions outside the image hold dx/dy of the remapped pixel
    if (!(x0 - 1 >= 0 && x0 + TW < w && y0 - 1 >= 0 && y0 + TH < h)) {
        __syncthreads();
        for (int k = tid; k < EH * EW; k += TW) {
            const int r = k / EW, c = k % EW;
            const int gx = x0 - 1 + c, gy = y0 - 1 + r;
            if (gx >= 0 && gx < w && gy >= 0 && gy < h) continue;
            int vx, vy;
            if (p.mode == ISP_CONSTANT) {
                vx = vy = p.hcval;
            } else {
                const int bx = bmap(p.mode, gx, w), by = bmap(p.mode, gy, h);
                int t[3][3];
#pragma unroll
                for (int j = 0; j < 3; ++j)
#pragma unroll
                    for (int i = 0; i < 3; ++i)
                        t[j][i] = rd_img(p.img, w, h, p.pitch, p.mode, p.cval, bx + i - 1, by + j - 1);
                vx = (t[0][2] - t[0][0]) + 2 * (t[1][2] - t[1][0]) + (t[2][2] - t[2][0]);
                vy = (t[2][0] + 2 * t[2][1] + t[2][2]) - (t[0][0] + 2 * t[0][1] + t[0][2]);
            }
            s_dx[r][c] = (int16_t)vx;
            s_dy[r][c] = (int16_t)vy;
        }
    }
    __syncthreads();

    // ---- outputs: thread = column x0+tid, walk rows y0 .. y0+TH-1 -------------------------
    const int x = x0 + tid;
    if (x >= w) return;
    const int sc = XO + tid;  // s_in column of x
    const int ec = tid + 1;   // ext column of x
    const int ylast = min(TH, h - y0);
    const double thr = (double)max(-9007199254740992ll, min(9007199254740992ll, p.thr));

    // Laplace ring of horizontal 5-sums (s_in rows r .. r+4 for output row r)
    int b0, b1, b2, b3;
    auto box = [&](int r) {
        return (int)s_in[r][sc - 2] + s_in[r][sc - 1] + s_in[r][sc] + s_in[r][sc + 1] + s_in[r][sc + 2];
    };
    b0 = box(0); b1 = box(1); b2 = box(2); b3 = box(3);
    // Harris ring of horizontal weighted sums (ext rows r .. r+2 for output row r)
    int hxx0, hyy0, hxy0, hxx1, hyy1, hxy1;
    auto hsum = [&](int r, int &xx, int &yy, int &xy) {
        const int gx0 = s_dx[r][ec - 1], gx1 = s_dx[r][ec], gx2 = s_dx[r][ec + 1];
        const int gy0 = s_dy[r][ec - 1], gy1 = s_dy[r][ec], gy2 = s_dy[r][ec + 1];
        xx = gx0 * gx0 + 2 * gx1 * gx1 + gx2 * gx2;
        yy = gy0 * gy0 + 2 * gy1 * gy1 + gy2 * gy2;
        xy = gx0 * gy0 + 2 * gx1 * gy1 + gx2 * gy2;
    };
    hsum(0, hxx0, hyy0, hxy0);
    hsum(1, hxx1, hyy1, hxy1);

#pragma unroll 4
    for (int r = 0; r < TH; ++r) {
        if (r >= ylast) break;
        const size_t off = (size_t)(y0 + r) * p.out_pitch + x;
        // Sobel
        const int gx = s_dx[r + 1][ec], gy = s_dy[r + 1][ec];
        p.mag[off] = (uint8_t)mag_u8(gx * gx + gy * gy);
        if (p.dx) p.dx[off] = (int16_t)gx;
        if (p.dy) p.dy[off] = (int16_t)gy;
        // Laplace: sum of 25 minus 25 x centre
        const int b4 = box(r + 4);
        const int acc = b0 + b1 + b2 + b3 + b4 - 25 * (int)s_in[r + 2][sc];
        p.lap[off] = (uint8_t)min(255, max(0, acc));
        b0 = b1; b1 = b2; b2 = b3; b3 = b4;
        // Harris: Sxx etc. < 2^24 in magnitude (int32 exact); response exact in f64
        int hxx2, hyy2, hxy2;
        hsum(r + 2, hxx2, hyy2, hxy2);
        const int sxx = hxx0 + 2 * hxx1 + hxx2, syy = hyy0 + 2 * hyy1 + hyy2, sxy = hxy0 + 2 * hxy1 + hxy2;
        const double dxx = sxx, dyy = syy, dxy = sxy;
        const double det = fma(-dxy, dxy, dxx * dyy);
        const double tr = dxx + dyy;
        const double r25 = fma(25.0, det, -(tr * tr));
        p.har[off] = r25 > thr ? 255 : 0;
        hxx0 = hxx1; hyy0 = hyy1; hxy0 = hxy1;
        hxx1 = hxx2; hyy1 = hyy2; hxy1 = hxy2;
    }
}

size_t span(int w, int h, int pitch, size_t es) { return ((size_t)(h - 1) * pitch + w) * es; }
bool overlap(const void *a, size_t na, const void *b, size_t nb)
{
    const char *x = (const char *)a, *y = (const char *)b;
    return x < y + nb && y < x + na;
}

}  // namespace

extern "C" isp_status_t isp_pipeline_cfg3_u8(const uint8_t *img, int w, int h, int pitch, int border_mode,
                                             int const_val, int harris_const, int64_t thr, int16_t *dx,
                                             int16_t *dy, uint8_t *mag, uint8_t *lap, uint8_t *harris,
                                             int out_pitch, isp_variant_t variant, isp_stream_t stream)
{
    if (w < 1 || h < 1) return ispi_fail(ISP_EINVAL, "image size %dx%d", w, h);
    if (pitch < w || out_pitch < w) return ispi_fail(ISP_EINVAL, "pitch %d / out_pitch %d < width %d", pitch, out_pitch, w);
    if (border_mode < 0 || border_mode > 3) return ispi_fail(ISP_EINVAL, "border mode %d", border_mode);
    if (!img || !mag || !lap || !harris) return ispi_fail(ISP_EINVAL, "null pointer");
    if (const_val < 0 || const_val > 255) return ispi_fail(ISP_EINVAL, "u8 constant %d not in [0,255]", const_val);
    if (harris_const < -1020 || harris_const > 1020)  // the range of Sobel derivatives: int32 sums stay exact
        return ispi_fail(ISP_EINVAL, "Harris constant %d not in [-1020,1020]", harris_const);
    if ((int)variant < 0 || (int)variant > 4) return ispi_fail(ISP_EINVAL, "variant %d", (int)variant);
    const size_t ib = span(w, h, pitch, 1), ob1 = span(w, h, out_pitch, 1), ob2 = span(w, h, out_pitch, 2);
    if (overlap(img, ib, mag, ob1) || overlap(img, ib, lap, ob1) || overlap(img, ib, harris, ob1) ||
        (dx && overlap(img, ib, dx, ob2)) || (dy && overlap(img, ib, dy, ob2)))
        return ispi_fail(ISP_EALIAS, "input and output overlap");
    if ((long long)w + 2 * XO > (1LL << 30) || (long long)h + 4 > (1LL << 30))
        return ispi_fail(ISP_EINVAL, "image too large");
    Params p;
    p.img = img;
    p.w = w; p.h = h; p.pitch = pitch; p.mode = border_mode;
    p.cval = const_val; p.hcval = harris_const; p.out_pitch = out_pitch;
    p.naive = variant == ISP_NAIVE;
    p.vec = ((uintptr_t)img % 16 == 0) && (pitch % 16 == 0);
    p.thr = thr;
    p.dx = dx; p.dy = dy; p.mag = mag; p.lap = lap; p.har = harris;
    const dim3 grid((w + TW - 1) / TW, (h + TH - 1) / TH);
    k_fused_cfg3<<<grid, TW, 0, (cudaStream_t)stream>>>(p);
    const cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return ispi_fail(ISP_ECUDA, "isp_pipeline_cfg3_u8: %s", cudaGetErrorString(e));
    return ISP_OK;
}
