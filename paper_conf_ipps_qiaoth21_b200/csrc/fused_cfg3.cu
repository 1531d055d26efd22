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
// CTA = 128 threads, tile 128x32: each lane owns 4 adjacent columns (word-wide shared
// loads, packed 4-byte stores), each warp 16 rows walked with register rings.
#include <cuda_runtime.h>
#include <stdint.h>

#include <cstring>

#include "../../include/isp.h"
#include "internal.h"

namespace {

constexpr int NT = 128;                // threads per CTA
constexpr int TW = 128;                // output columns per CTA (32 lanes x 4 pixels)
#ifndef FUSED_TH
#define FUSED_TH 32
#endif
#ifndef FUSED_MINB
#define FUSED_MINB 4
#endif
// Row loops are kept rolled: fully unrolled, the kernel's hot code (~43 KB of SASS) missed
// the instruction cache ("no_instructions" was the top stall in the ncu capture).
#ifndef FUSED_UNROLL_R
#define FUSED_UNROLL_R 1
#endif
#ifndef FUSED_UNROLL_E
#define FUSED_UNROLL_E 1
#endif
constexpr int kUnrollR = FUSED_UNROLL_R, kUnrollE = FUSED_UNROLL_E;
constexpr int TH = FUSED_TH;           // output rows per CTA (4 warps x TH/4 rows)
constexpr int RPW = TH / (NT / 32);    // rows per warp
constexpr int XO = 16;                 // staged input starts at x0 - XO (16-byte aligned)
constexpr int SW = TW + 2 * XO;        // staged row width (bytes)
constexpr int SH = TH + 4;             // staged rows: y0-2 .. y0+TH+1
constexpr int EW = TW + 2, EH = TH + 2;  // dx/dy ext: x0-1 .. x0+TW, y0-1 .. y0+TH
constexpr int EWS = TW + 4;            // ext row stride (int16), multiple of 4
constexpr int NG = (EW + 3) / 4;       // 4-column groups of the ext grid
constexpr int NSEG = NT / NG, SEGR = (EH + NSEG - 1) / NSEG;  // one item per thread

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

// min(255, round_half_up(sqrt(n))) (a9) for 0 <= n: n is clamped to 65280 = 255.5^2 - 1/4
// (larger n saturate), sqrt.approx errs by < 1e-4 there while the nearest half-integer
// is >= 1/(2*511) away for integer n -- the proof in DESIGN.md section 7c (`sobel_mag`).
__device__ __forceinline__ int mag_u8(int n)
{
    const float f = (float)min(n, 65280);
    float r;
    asm("sqrt.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(f));
    return (int)(r + 0.5f);
}

__device__ __forceinline__ int byte_of(uint32_t v, int k) { return (v >> (8 * k)) & 0xff; }
__device__ __forceinline__ int lo16(uint32_t v) { return (int)(int16_t)(v & 0xffff); }
__device__ __forceinline__ int hi16(uint32_t v) { return (int)v >> 16; }
__device__ __forceinline__ uint32_t pack16(int a, int b) { return (uint32_t)(uint16_t)a | ((uint32_t)(uint16_t)b << 16); }

struct Params;
__device__ __noinline__ void fix_ext(const Params &p, int gx, int gy, int16_t *ox, int16_t *oy);
__device__ __noinline__ void store_tail(const Params &p, size_t off, int x, const int (&lap)[4], const int (&har)[4],
                                        const int (&mag)[4], const int (&cx)[4], const int (&cy)[4]);

struct Params {
    const uint8_t *img;
    int w, h, pitch, mode, cval, hcval, out_pitch, naive, vec, vec_out;
    long long thr;
    int16_t *dx, *dy;
    uint8_t *mag, *lap, *har;
};

__global__ void __launch_bounds__(NT, FUSED_MINB) k_fused_cfg3(const Params p)
{
    __shared__ __align__(16) uint8_t s_in[SH][SW];
    __shared__ __align__(16) int16_t s_dx[EH][EWS];
    __shared__ __align__(16) int16_t s_dy[EH][EWS];

    const int tid = threadIdx.x;
    const int x0 = blockIdx.x * TW, y0 = blockIdx.y * TH;
    const int w = p.w, h = p.h;

    // ---- stage img(B(x), B(y)) for x in [x0-2, x0+TW+2), y in [y0-2, y0+TH+2) ----------
    const bool body = !p.naive && p.vec && x0 - XO >= 0 && x0 + TW + XO <= w && y0 - 2 >= 0 && y0 + TH + 2 <= h;
    if (body) {
        constexpr int VPR = SW / 16;
        for (int k = tid; k < SH * VPR; k += NT) {
            const int r = k / VPR, c = k % VPR;
            const uint4 v = __ldg(reinterpret_cast<const uint4 *>(p.img + (size_t)(y0 - 2 + r) * p.pitch + x0 - XO) + c);
            *reinterpret_cast<uint4 *>(&s_in[r][c * 16]) = v;
        }
    } else {
        constexpr int GW = TW + 4;
        for (int k = tid; k < SH * GW; k += NT) {
            const int r = k / GW, c = k % GW;
            s_in[r][XO - 2 + c] = (uint8_t)rd_img(p.img, w, h, p.pitch, p.mode, p.cval, x0 - 2 + c, y0 - 2 + r);
        }
    }
    __syncthreads();

    // ---- dx, dy on the ext grid: ext column e <-> x0-1+e, ext row er <-> y0-1+er ----------
    // 4 ext columns per item, a row segment walked with a 3-row register ring.
    for (int it = tid; it < NG * NSEG; it += NT) {
        const int e0 = 4 * (it % NG), rs = (it / NG) * SEGR, re = min(EH, rs + SEGR);
        int d0[4], d1[4], s0[4], s1[4];
        auto hrow = [&](int srow, int (&d)[4], int (&sm)[4]) {
            // s_in columns XO+e0-2 .. XO+e0+3 (rel -2..3) from two aligned words
            const uint32_t a = *reinterpret_cast<const uint32_t *>(&s_in[srow][XO + e0 - 4]);
            const uint32_t b = *reinterpret_cast<const uint32_t *>(&s_in[srow][XO + e0]);
            const int v[6] = {byte_of(a, 2), byte_of(a, 3), byte_of(b, 0), byte_of(b, 1), byte_of(b, 2), byte_of(b, 3)};
#pragma unroll
            for (int k = 0; k < 4; ++k) {
                d[k] = v[k + 2] - v[k];
                sm[k] = v[k] + 2 * v[k + 1] + v[k + 2];
            }
        };
        hrow(rs, d0, s0);      // ext row er has s_in rows er .. er+2
        hrow(rs + 1, d1, s1);
#pragma unroll(kUnrollE)
        for (int i = 0; i < SEGR; ++i) {
            const int er = rs + i;
            if (er >= re) break;
            int d2[4], s2[4];
            hrow(er + 2, d2, s2);
            int gx[4], gy[4];
#pragma unroll
            for (int k = 0; k < 4; ++k) {
                gx[k] = d0[k] + 2 * d1[k] + d2[k];
                gy[k] = s2[k] - s0[k];
                d0[k] = d1[k]; d1[k] = d2[k]; s0[k] = s1[k]; s1[k] = s2[k];
            }
            *reinterpret_cast<uint2 *>(&s_dx[er][e0]) = make_uint2(pack16(gx[0], gx[1]), pack16(gx[2], gx[3]));
            *reinterpret_cast<uint2 *>(&s_dy[er][e0]) = make_uint2(pack16(gy[0], gy[1]), pack16(gy[2], gy[3]));
        }
    }
    // border tiles: ext positions outside the image hold dx/dy of the remapped pixel
    if (!(x0 - 1 >= 0 && x0 + TW < w && y0 - 1 >= 0 && y0 + TH < h)) {
        __syncthreads();
        for (int k = tid; k < EH * EW; k += NT) {
            const int r = k / EW, c = k % EW;
            const int gx = x0 - 1 + c, gy = y0 - 1 + r;
            if (gx >= 0 && gx < w && gy >= 0 && gy < h) continue;
            fix_ext(p, gx, gy, &s_dx[r][c], &s_dy[r][c]);
        }
    }
    __syncthreads();

    // ---- outputs: lane -> 4 columns, warp -> RPW rows, register rings down the rows ------
    const int xr = 4 * (tid & 31);
    const int x = x0 + xr;
    const int rbeg = (tid >> 5) * RPW;
    const int rend = min(rbeg + RPW, h - y0);
    if (x >= w || rbeg >= rend) return;
    const double thr = (double)max(-9007199254740992ll, min(9007199254740992ll, p.thr));
    const bool vec = p.vec_out && x + 3 < w;

    // Laplace: horizontal 5-sums of s_in row `sr` for the 4 pixels (rel -2..5)
    auto box4 = [&](int sr, int (&bx)[4]) {
        const uint32_t a = *reinterpret_cast<const uint32_t *>(&s_in[sr][XO + xr - 4]);
        const uint32_t b = *reinterpret_cast<const uint32_t *>(&s_in[sr][XO + xr]);
        const uint32_t c = *reinterpret_cast<const uint32_t *>(&s_in[sr][XO + xr + 4]);
        const int v[8] = {byte_of(a, 2), byte_of(a, 3), byte_of(b, 0), byte_of(b, 1),
                          byte_of(b, 2), byte_of(b, 3), byte_of(c, 0), byte_of(c, 1)};
        bx[0] = v[0] + v[1] + v[2] + v[3] + v[4];
        bx[1] = bx[0] - v[0] + v[5];
        bx[2] = bx[1] - v[1] + v[6];
        bx[3] = bx[2] - v[2] + v[7];
    };
    // Harris: horizontal [1,2,1] sums of the products on ext row `er` (ext cols xr .. xr+5);
    // also returns the row's own dx/dy at the 4 pixels (ext cols xr+1 .. xr+4).
    auto hsum4 = [&](int er, int (&hxx)[4], int (&hyy)[4], int (&hxy)[4], int (&cx)[4], int (&cy)[4]) {
        const uint2 ax = *reinterpret_cast<const uint2 *>(&s_dx[er][xr]);
        const uint32_t bx = *reinterpret_cast<const uint32_t *>(&s_dx[er][xr + 4]);
        const uint2 ay = *reinterpret_cast<const uint2 *>(&s_dy[er][xr]);
        const uint32_t by = *reinterpret_cast<const uint32_t *>(&s_dy[er][xr + 4]);
        const int gx[6] = {lo16(ax.x), hi16(ax.x), lo16(ax.y), hi16(ax.y), lo16(bx), hi16(bx)};
        const int gy[6] = {lo16(ay.x), hi16(ay.x), lo16(ay.y), hi16(ay.y), lo16(by), hi16(by)};
        int pxx[6], pyy[6], pxy[6];
#pragma unroll
        for (int i = 0; i < 6; ++i) {
            pxx[i] = gx[i] * gx[i];
            pyy[i] = gy[i] * gy[i];
            pxy[i] = gx[i] * gy[i];
        }
#pragma unroll
        for (int k = 0; k < 4; ++k) {
            hxx[k] = pxx[k] + 2 * pxx[k + 1] + pxx[k + 2];
            hyy[k] = pyy[k] + 2 * pyy[k + 1] + pyy[k + 2];
            hxy[k] = pxy[k] + 2 * pxy[k + 1] + pxy[k + 2];
            cx[k] = gx[k + 1];
            cy[k] = gy[k + 1];
        }
    };

    int B0[4], B1[4], B2[4], B3[4];
    box4(rbeg, B0); box4(rbeg + 1, B1); box4(rbeg + 2, B2); box4(rbeg + 3, B3);
    int X0[4], Y0[4], Z0[4], X1[4], Y1[4], Z1[4], cx0[4], cy0[4], cx1[4], cy1[4];
    hsum4(rbeg, X0, Y0, Z0, cx0, cy0);
    hsum4(rbeg + 1, X1, Y1, Z1, cx1, cy1);

#pragma unroll(kUnrollR)
    for (int i = 0; i < RPW; ++i) {
        const int r = rbeg + i;
        if (r >= rend) break;
        const size_t off = (size_t)(y0 + r) * p.out_pitch + x;
        // Laplace: five box rows minus 25 x centre (s_in row r+2)
        int B4[4];
        box4(r + 4, B4);
        const uint32_t cw = *reinterpret_cast<const uint32_t *>(&s_in[r + 2][XO + xr]);
        int lap[4];
#pragma unroll
        for (int k = 0; k < 4; ++k) {
            lap[k] = min(255, max(0, B0[k] + B1[k] + B2[k] + B3[k] + B4[k] - 25 * byte_of(cw, k)));
            B0[k] = B1[k]; B1[k] = B2[k]; B2[k] = B3[k]; B3[k] = B4[k];
        }
        // Harris (exact: window sums < 2^24, response in f64) and Sobel on ext row r+1
        int X2[4], Y2[4], Z2[4], cx2[4], cy2[4];
        hsum4(r + 2, X2, Y2, Z2, cx2, cy2);
        int har[4], mag[4];
#pragma unroll
        for (int k = 0; k < 4; ++k) {
            const double sxx = X0[k] + 2 * X1[k] + X2[k], syy = Y0[k] + 2 * Y1[k] + Y2[k];
            const double sxy = Z0[k] + 2 * Z1[k] + Z2[k];
            const double det = fma(-sxy, sxy, sxx * syy);
            const double tr = sxx + syy;
            har[k] = fma(25.0, det, -(tr * tr)) > thr ? 255 : 0;
            mag[k] = mag_u8(cx1[k] * cx1[k] + cy1[k] * cy1[k]);
        }
        if (vec) {
            *reinterpret_cast<uint32_t *>(p.lap + off) = lap[0] | lap[1] << 8 | lap[2] << 16 | lap[3] << 24;
            *reinterpret_cast<uint32_t *>(p.har + off) = har[0] | har[1] << 8 | har[2] << 16 | har[3] << 24;
            *reinterpret_cast<uint32_t *>(p.mag + off) = mag[0] | mag[1] << 8 | mag[2] << 16 | mag[3] << 24;
            if (p.dx) *reinterpret_cast<uint2 *>(p.dx + off) = make_uint2(pack16(cx1[0], cx1[1]), pack16(cx1[2], cx1[3]));
            if (p.dy) *reinterpret_cast<uint2 *>(p.dy + off) = make_uint2(pack16(cy1[0], cy1[1]), pack16(cy1[2], cy1[3]));
        } else {
            store_tail(p, off, x, lap, har, mag, cx1, cy1);
        }
#pragma unroll
        for (int k = 0; k < 4; ++k) {
            X0[k] = X1[k]; Y0[k] = Y1[k]; Z0[k] = Z1[k];
            X1[k] = X2[k]; Y1[k] = Y2[k]; Z1[k] = Z2[k];
            cx1[k] = cx2[k]; cy1[k] = cy2[k];
        }
    }
    (void)cx0; (void)cy0;
}

// Cold paths kept out of line (instruction-cache footprint of the hot loop).
// dx/dy of the dx/dy IMAGES at an ext position outside the image: the Sobel value at the
// remapped pixel B(gx), B(gy); Constant: the Harris constant.
__device__ __noinline__ void fix_ext(const Params &p, int gx, int gy, int16_t *ox, int16_t *oy)
{
    int vx, vy;
    if (p.mode == ISP_CONSTANT) {
        vx = vy = p.hcval;
    } else {
        const int bx = bmap(p.mode, gx, p.w), by = bmap(p.mode, gy, p.h);
        int t[3][3];
        for (int j = 0; j < 3; ++j)
            for (int i = 0; i < 3; ++i)
                t[j][i] = rd_img(p.img, p.w, p.h, p.pitch, p.mode, p.cval, bx + i - 1, by + j - 1);
        vx = (t[0][2] - t[0][0]) + 2 * (t[1][2] - t[1][0]) + (t[2][2] - t[2][0]);
        vy = (t[2][0] + 2 * t[2][1] + t[2][2]) - (t[0][0] + 2 * t[0][1] + t[0][2]);
    }
    *ox = (int16_t)vx;
    *oy = (int16_t)vy;
}

// Element-wise stores for the image's last partial column group or unaligned outputs.
__device__ __noinline__ void store_tail(const Params &p, size_t off, int x, const int (&lap)[4], const int (&har)[4],
                                        const int (&mag)[4], const int (&cx)[4], const int (&cy)[4])
{
    for (int k = 0; k < 4 && x + k < p.w; ++k) {
        p.lap[off + k] = (uint8_t)lap[k];
        p.har[off + k] = (uint8_t)har[k];
        p.mag[off + k] = (uint8_t)mag[k];
        if (p.dx) p.dx[off + k] = (int16_t)cx[k];
        if (p.dy) p.dy[off + k] = (int16_t)cy[k];
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
    p.vec_out = out_pitch % 4 == 0 && (uintptr_t)mag % 4 == 0 && (uintptr_t)lap % 4 == 0 &&
                (uintptr_t)harris % 4 == 0 && (!dx || (uintptr_t)dx % 8 == 0) && (!dy || (uintptr_t)dy % 8 == 0);
    p.thr = thr;
    p.dx = dx; p.dy = dy; p.mag = mag; p.lap = lap; p.har = harris;
    const dim3 grid((w + TW - 1) / TW, (h + TH - 1) / TH);
    k_fused_cfg3<<<grid, NT, 0, (cudaStream_t)stream>>>(p);
    const cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return ispi_fail(ISP_ECUDA, "isp_pipeline_cfg3_u8: %s", cudaGetErrorString(e));
    return ISP_OK;
}
