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

#include <algorithm>
#include <cstdlib>
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
    // tile-ISP kernel (round 2): tiles [bx0, bx1) x [by0, by1) are its Body region
    int nbx, nby, bx0, bx1, by0, by1;
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

// =====================================================================================
// Body-tile kernel (round 2).  Runs only tiles whose whole staged window lies inside the
// image (the Body region of the tile partition, Listing 3 at tile granularity): no checks,
// no remapped ext positions, so it can be built for instruction count and occupancy:
//   * Sobel's horizontal parts on 16-bit pair lanes (SWAR: pixels (0,2) and (1,3) of a
//     4-pixel group share one 32-bit register; all lanes stay in [0, 65535], biased where
//     a value can be negative, so no carry / borrow crosses lanes);
//   * the dx / dy ext grid in shared memory as exact floats (|dx|, |dy| <= 1020);
//   * Harris window sums with packed FP32x2 FMAs (exact: integers < 2^24), the response
//     in f32 with a rigorous error bound and the exact f64 evaluation only when the bound
//     cannot decide R25 > thr;
//   * Laplace horizontal 5-sums with DP4A on byte windows, vertical sums in a 5-row ring.
// Output bits equal the general kernel's (and the oracle composition's).
// =====================================================================================
constexpr int G2 = 34;                                  // ext groups: cols x0-4+4G .. x0-1+4G
constexpr int EWF = 4 * G2;                             // floats per ext row
constexpr int NSEG2 = NT / G2, SEGR2 = (EH + NSEG2 - 1) / NSEG2;
#ifndef FUSED_BODY_MINB
#define FUSED_BODY_MINB 5
#endif

struct BodySmem {
    uint8_t in[SH][SW];                                 // image rows y0-2.., cols x0-16..
    float fx[EH][EWF], fy[EH][EWF];                     // per group [p0, p2, p1, p3]
};

__device__ __forceinline__ uint32_t lw(const uint8_t *p) { return *reinterpret_cast<const uint32_t *>(p); }

// 16-bit lanes (biased by 1024) -> exact floats: 2^23 + lane has the lane in its mantissa
__device__ __forceinline__ float2 lanes_f(uint32_t x)
{
    const float b = 8388608.0f + 1024.0f;
    return make_float2(__uint_as_float(__byte_perm(x, 0x4B000000u, 0x7610)) - b,
                       __uint_as_float(__byte_perm(x, 0x4B000000u, 0x7632)) - b);
}

// Sobel horizontal parts of one staged row for the 4 pixels at s_in column c (pairs:
// E = pixels (0, 2), O = (1, 3)): s = a + 2b + c, d = c - a + 256 (bias).
__device__ __forceinline__ void hsob(const uint8_t *row, int c, uint32_t &sE, uint32_t &sO, uint32_t &dE,
                                     uint32_t &dO)
{
    const uint32_t A = lw(row + c - 4), B = lw(row + c), C = lw(row + c + 4);
    const uint32_t Ec = __byte_perm(B, 0u, 0x4240), Oc = __byte_perm(B, 0u, 0x4341);
    const uint32_t El = __byte_perm(A, B, 0x0503) & 0x00FF00FFu;   // (c-1, c1)
    const uint32_t Or = __byte_perm(B, C, 0x0402) & 0x00FF00FFu;   // (c2, c4)
    sE = El + 2u * Ec + Oc;
    sO = Ec + 2u * Oc + Or;
    dE = Oc + 0x01000100u - El;
    dO = Or + 0x01000100u - Ec;
}

__device__ __forceinline__ float2 f2(float a, float b) { return make_float2(a, b); }
__device__ __forceinline__ float2 mul2(float2 a, float2 b)
{
    unsigned long long x, y, z;
    asm("mov.b64 %0, {%1, %2};" : "=l"(x) : "f"(a.x), "f"(a.y));
    asm("mov.b64 %0, {%1, %2};" : "=l"(y) : "f"(b.x), "f"(b.y));
    asm("mul.rn.f32x2 %0, %1, %2;" : "=l"(z) : "l"(x), "l"(y));
    float2 r;
    asm("mov.b64 {%0, %1}, %2;" : "=f"(r.x), "=f"(r.y) : "l"(z));
    return r;
}
__device__ __forceinline__ float2 fma2(float2 a, float2 b, float2 c)
{
    unsigned long long x, y, z, w;
    asm("mov.b64 %0, {%1, %2};" : "=l"(x) : "f"(a.x), "f"(a.y));
    asm("mov.b64 %0, {%1, %2};" : "=l"(y) : "f"(b.x), "f"(b.y));
    asm("mov.b64 %0, {%1, %2};" : "=l"(z) : "f"(c.x), "f"(c.y));
    asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(w) : "l"(x), "l"(y), "l"(z));
    float2 r;
    asm("mov.b64 {%0, %1}, %2;" : "=f"(r.x), "=f"(r.y) : "l"(w));
    return r;
}
__device__ __forceinline__ float2 add2(float2 a, float2 b)
{
    unsigned long long x, y, z;
    asm("mov.b64 %0, {%1, %2};" : "=l"(x) : "f"(a.x), "f"(a.y));
    asm("mov.b64 %0, {%1, %2};" : "=l"(y) : "f"(b.x), "f"(b.y));
    asm("add.rn.f32x2 %0, %1, %2;" : "=l"(z) : "l"(x), "l"(y));
    float2 r;
    asm("mov.b64 {%0, %1}, %2;" : "=f"(r.x), "=f"(r.y) : "l"(z));
    return r;
}

// Horizontal [1,2,1] sums of xx, yy, xy over ext row e for the 4 pixels of group G, as
// pairs (H(p0), H(p2)) and (H(p1), H(p3)).  Exact: integer products / sums < 2^24.
struct HS { float2 xxE, xxO, yyE, yyO, xyE, xyO; };
__device__ __forceinline__ HS hsum_row(const float *fxr, const float *fyr, int G)
{
    const float4 X = *reinterpret_cast<const float4 *>(fxr + 4 * G);     // p0, p2, p1, p3
    const float4 Y = *reinterpret_cast<const float4 *>(fyr + 4 * G);
    const float xl = fxr[4 * G - 1], yl = fyr[4 * G - 1];                 // p-1 (left group's p3)
    const float xr = fxr[4 * G + 4], yr = fyr[4 * G + 4];                 // p4 (right group's p0)
    const float2 xE = f2(X.x, X.y), xO = f2(X.z, X.w), yE = f2(Y.x, Y.y), yO = f2(Y.z, Y.w);
    // products at positions: E = (p0, p2), O = (p1, p3), A = (p-1, p1), B = (p2, p4)
    const float2 xxE = mul2(xE, xE), xxO = mul2(xO, xO), yyE = mul2(yE, yE), yyO = mul2(yO, yO);
    const float2 xyE = mul2(xE, yE), xyO = mul2(xO, yO);
    const float2 xxA = f2(xl * xl, xxO.x), xxB = f2(xxE.y, xr * xr);
    const float2 yyA = f2(yl * yl, yyO.x), yyB = f2(yyE.y, yr * yr);
    const float2 xyA = f2(xl * yl, xyO.x), xyB = f2(xyE.y, xr * yr);
    const float2 two = f2(2.f, 2.f);
    HS h;
    h.xxE = add2(fma2(two, xxE, xxA), xxO);   // (H0, H2) = A + 2E + O
    h.xxO = add2(fma2(two, xxO, xxE), xxB);   // (H1, H3) = E + 2O + B
    h.yyE = add2(fma2(two, yyE, yyA), yyO);
    h.yyO = add2(fma2(two, yyO, yyE), yyB);
    h.xyE = add2(fma2(two, xyE, xyA), xyO);
    h.xyO = add2(fma2(two, xyO, xyE), xyB);
    return h;
}

// Exact R25 > thr (f64: every intermediate is an integer < 2^53).
__device__ __noinline__ int harris_exact(float sxx, float syy, float sxy, double thr)
{
    const double dx = sxx, dy = syy, dz = sxy;
    const double dd = fma(-dz, dz, dx * dy), tr = dx + dy;
    return fma(25.0, dd, -(tr * tr)) > thr ? 255 : 0;
}

// R25 > thr for a pair of pixels from exact window sums (floats, integers < 2^24).
// Fast f32 path: |R_f - R| <= 2^-17 (p + q + t^2) (generous bound on five roundings,
// DESIGN.md 7g); a pixel the bound cannot decide takes the exact f64 evaluation (out of
// line; all sums zero -- a flat area -- means R25 = 0 exactly).
__device__ __forceinline__ void harris2(float2 sxx, float2 syy, float2 sxy, float thr_f, float thr_err, double thr,
                                        int &o0, int &o1)
{
    const float2 p = mul2(sxx, syy), q = mul2(sxy, sxy);
    const float2 det = fma2(f2(-sxy.x, -sxy.y), sxy, p);
    const float2 t = add2(sxx, syy);
    const float2 tt = mul2(t, t);
    const float2 R = fma2(f2(25.f, 25.f), det, f2(-tt.x, -tt.y));
    const float2 bnd = add2(add2(p, q), tt);
    // (1 + 2^-10) x the bound: |d| >= b decides strictly (b = 0: flat area, thr = 0, exact)
    const float b0 = fmaf(bnd.x, 7.6368451118469238281e-06f, thr_err), b1 = fmaf(bnd.y, 7.6368451118469238281e-06f, thr_err);
    const float d0 = R.x - thr_f, d1 = R.y - thr_f;
    o0 = d0 > 0.f ? 255 : 0;
    o1 = d1 > 0.f ? 255 : 0;
    const bool u0 = fabsf(d0) < b0, u1 = fabsf(d1) < b1;     // undecided by the bound
    if (__any_sync(0xffffffffu, u0 || u1)) {
        if (u0) o0 = bnd.x == 0.f ? (0.0 > thr ? 255 : 0) : harris_exact(sxx.x, syy.x, sxy.x, thr);
        if (u1) o1 = bnd.y == 0.f ? (0.0 > thr ? 255 : 0) : harris_exact(sxx.y, syy.y, sxy.y, thr);
    }
}

__device__ __forceinline__ int mag_f(float n)
{
    float r;
    asm("sqrt.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(fminf(n, 65280.0f)));
    return (int)(r + 0.5f);
}

// Border pattern for an overshoot below N (one reflection / wrap): the tile-ISP launch
// only runs on images of at least 2 x 2 tiles, whose staged windows reach 16 columns and
// 2 rows past the edge.
__device__ __forceinline__ int bmap1(int mode, int i, int n)
{
    if (i >= 0 && i < n) return i;
    switch (mode) {
    case ISP_CLAMP: return i < 0 ? 0 : n - 1;
    case ISP_MIRROR: return i < 0 ? -i - 1 : 2 * n - 1 - i;
    case ISP_REPEAT: return i < 0 ? i + n : i - n;
    default: return -1;
    }
}

// Border tile staging: rows through the pattern once per row; 16-byte vectors whose columns
// are all inside the image are copied as vectors, the rest byte by byte through the pattern
// (the Body-tile launch requires w, h >= 2 tiles, so overshoots stay below N).
__device__ __noinline__ void stage_border(const Params &p, uint8_t *in, int x0, int y0)
{
    constexpr int VPR = SW / 16;
    for (int k = threadIdx.x; k < SH * VPR; k += NT) {
        const int r = k / VPR, c = k % VPR;
        const int yy = bmap1(p.mode, y0 - 2 + r, p.h);         // -1: Constant, row outside
        uint8_t *dst = in + r * SW + 16 * c;
        const int xs = x0 - XO + 16 * c;
        if (yy >= 0 && xs >= 0 && xs + 16 <= p.w) {
            *reinterpret_cast<uint4 *>(dst) = __ldg(reinterpret_cast<const uint4 *>(p.img + (size_t)yy * p.pitch + xs));
        } else {
            for (int e = 0; e < 16; ++e) {
                const int xx = bmap1(p.mode, xs + e, p.w);
                dst[e] = (uint8_t)((yy < 0 || xx < 0) ? p.cval : p.img[(size_t)yy * p.pitch + xx]);
            }
        }
    }
}

// Ext grid positions the stored outputs read that lie outside the image (x = -1 or w,
// y = -1 or h): the Sobel value of the remapped pixel (or the Harris constant).
__device__ __forceinline__ int ext_slot(int gx, int x0)   // ext column slot of image column gx
{
    const int rel = gx - (x0 - 4), G = rel >> 2, pos = rel & 3;   // slots hold p0, p2, p1, p3
    return 4 * G + (pos == 0 ? 0 : pos == 1 ? 2 : pos == 2 ? 1 : 3);
}

__device__ __noinline__ void fix_ext_border(const Params &p, float *fx, float *fy, int x0, int y0)
{
    const int w = p.w, h = p.h;
    auto fix = [&](int gx, int gy) {
        int16_t vx, vy;
        fix_ext(p, gx, gy, &vx, &vy);
        const int k = (gy - (y0 - 1)) * EWF + ext_slot(gx, x0);
        fx[k] = (float)vx;
        fy[k] = (float)vy;
    };
    // columns x = -1 and x = w (rows y in [-1, h])
    for (int k = threadIdx.x; k < 2 * EH; k += NT) {
        const int gy = y0 - 1 + (k >> 1), gx = (k & 1) ? w : -1;
        if (gx >= x0 - 4 && gx < x0 - 4 + EWF && gy >= -1 && gy <= h) fix(gx, gy);
    }
    // rows y = -1 and y = h (columns inside the image; the corners were done above)
    for (int k = threadIdx.x; k < 2 * EWF; k += NT) {
        const int gy = k < EWF ? -1 : h, gx = x0 - 4 + (k % EWF);
        if (gy >= y0 - 1 && gy < y0 - 1 + EH && gx >= 0 && gx < w) fix(gx, gy);
    }
}

// Tile order of the tile-ISP launch: the border tiles (slow: patterned staging, ext fix-ups)
// first, so they do not trail the last wave; then the Body tiles row-major.
__device__ __forceinline__ void tile_of(const Params &p, int k, int &bx, int &by)
{
    const int nb_in = (p.bx1 - p.bx0) * (p.by1 - p.by0), nframe = p.nbx * p.nby - nb_in;
    if (k >= nframe) {
        k -= nframe;
        const int iw = p.bx1 - p.bx0;
        bx = p.bx0 + k % iw;
        by = p.by0 + k / iw;
        return;
    }
    const int inner_w = p.bx1 - p.bx0, per_mid = p.nbx - inner_w;
    const int top = p.by0 * p.nbx, mid = (p.by1 - p.by0) * per_mid;
    if (k < top) { by = k / p.nbx; bx = k % p.nbx; return; }
    k -= top;
    if (k < mid) {
        by = p.by0 + k / per_mid;
        const int j = k % per_mid;
        bx = j < p.bx0 ? j : j + inner_w;
        return;
    }
    k -= mid;
    by = p.by1 + k / p.nbx;
    bx = k % p.nbx;
}

__global__ void __launch_bounds__(NT, FUSED_BODY_MINB) k_fused_body(const Params p)
{
    extern __shared__ __align__(16) unsigned char smem_raw[];
    BodySmem &S = *reinterpret_cast<BodySmem *>(smem_raw);
    const int tid = threadIdx.x;
    int bx, by;
    tile_of(p, (int)blockIdx.x, bx, by);
    const int x0 = bx * TW, y0 = by * TH;
    // Listing 3 at tile granularity: Body tiles read their whole window unchecked; border
    // tiles stage through the border pattern and fix up the ext positions outside the image
    const bool body = bx >= p.bx0 && bx < p.bx1 && by >= p.by0 && by < p.by1;

    // ---- stage img rows y0-2 .. y0+TH+1, cols x0-16 .. x0+TW+15 -------------------------
    if (body) {
        constexpr int VPR = SW / 16, DR = NT / VPR, DC = NT % VPR;   // (row, vector) stride per pass
        int r = tid / VPR, c = tid % VPR;
        const uint8_t *src = p.img + (size_t)(y0 - 2) * p.pitch + x0 - XO;
        for (; r < SH;) {
            *reinterpret_cast<uint4 *>(&S.in[r][c * 16]) = __ldg(reinterpret_cast<const uint4 *>(src + (size_t)r * p.pitch) + c);
            r += DR;
            c += DC;
            if (c >= VPR) { c -= VPR; ++r; }
        }
    } else {
        stage_border(p, &S.in[0][0], x0, y0);
    }
    __syncthreads();

    // ---- dx, dy on the ext grid (rows y0-1 .. y0+TH, cols x0-4 .. x0+TW+3) -------------
    for (int it = tid; it < G2 * NSEG2; it += NT) {
        const int G = it % G2, rs = (it / G2) * SEGR2, re = min(EH, rs + SEGR2);
        const int c = 12 + 4 * G;                           // s_in column of the group
        uint32_t sE0, sO0, dE0, dO0, sE1, sO1, dE1, dO1;
        hsob(S.in[rs], c, sE0, sO0, dE0, dO0);
        hsob(S.in[rs + 1], c, sE1, sO1, dE1, dO1);
        for (int er = rs; er < re; ++er) {
            uint32_t sE2, sO2, dE2, dO2;
            hsob(S.in[er + 2], c, sE2, sO2, dE2, dO2);
            const uint32_t dxE = dE0 + 2u * dE1 + dE2, dxO = dO0 + 2u * dO1 + dO2;   // + 1024 per lane
            const uint32_t dyE = sE2 + 0x04000400u - sE0, dyO = sO2 + 0x04000400u - sO0;
            const float2 xE = lanes_f(dxE), xO = lanes_f(dxO), yE = lanes_f(dyE), yO = lanes_f(dyO);
            *reinterpret_cast<float4 *>(&S.fx[er][4 * G]) = make_float4(xE.x, xE.y, xO.x, xO.y);
            *reinterpret_cast<float4 *>(&S.fy[er][4 * G]) = make_float4(yE.x, yE.y, yO.x, yO.y);
            sE0 = sE1; sO0 = sO1; dE0 = dE1; dO0 = dO1;
            sE1 = sE2; sO1 = sO2; dE1 = dE2; dO1 = dO2;
        }
    }
    if (!body) {   // ext positions outside the image: dx/dy of the remapped pixel (Harris' input)
        __syncthreads();
        fix_ext_border(p, &S.fx[0][0], &S.fy[0][0], x0, y0);
    }
    __syncthreads();

    // ---- outputs: lane -> 4 columns (group G = lane + 1), warp -> RPW rows ----------------
    const int lane = tid & 31, G = lane + 1;
    const int xr = 4 * lane, x = x0 + xr;
    const int rbeg = (tid >> 5) * RPW, rend = min(rbeg + RPW, p.h - y0);
    if (rbeg >= rend || x >= p.w) return;   // rows / columns past the image (partial tiles)
    const bool full = body || (x + 3 < p.w);
    const double thr = (double)max(-9007199254740992ll, min(9007199254740992ll, p.thr));
    const float thr_f = (float)thr;
    const float thr_err = 1.1932570487260818e-07f * fabsf(thr_f);   // |(float)thr - thr| x (1 + 2^-10)
    const uint32_t ones = 0x01010101u;
    // Laplace: horizontal 5-sums of staged row sr at the 4 pixels (DP4A on byte windows)
    auto h5 = [&](int sr, int (&H)[4]) {
        const uint8_t *row = S.in[sr] + XO + xr;
        const uint32_t L = lw(row - 4), B = lw(row), R = lw(row + 4);
        H[0] = (int)__dp4a(__funnelshift_r(L, B, 16), ones, (B >> 16) & 0xffu);
        H[1] = (int)__dp4a(__funnelshift_r(L, B, 24), ones, B >> 24);
        H[2] = (int)__dp4a(B, ones, R & 0xffu);
        H[3] = (int)__dp4a(__funnelshift_r(B, R, 8), ones, (R >> 8) & 0xffu);
    };
    int H0[4], H1[4], H2[4], H3[4];
    h5(rbeg, H0); h5(rbeg + 1, H1); h5(rbeg + 2, H2); h5(rbeg + 3, H3);
    HS a = hsum_row(S.fx[rbeg], S.fy[rbeg], G), b = hsum_row(S.fx[rbeg + 1], S.fy[rbeg + 1], G);
#pragma unroll 1
    for (int r = rbeg; r < rend; ++r) {
        const size_t off = (size_t)(y0 + r) * p.out_pitch + x;
        // Laplace (a8): box - 25 centre, clamped
        int H4[4];
        h5(r + 4, H4);
        const uint32_t cw = lw(S.in[r + 2] + XO + xr);
        // lap = clamp(box - 25 c, 0, 255) on 16-bit pair lanes: v = box + 25 (255 - c) is in
        // [0, 12750]; clamp to [6375, 6630] (u16x2 max / min), subtract 6375
        uint32_t bx_[4];
#pragma unroll
        for (int k = 0; k < 4; ++k) {
            bx_[k] = (uint32_t)(H0[k] + H1[k] + H2[k] + H3[k] + H4[k]);
            H0[k] = H1[k]; H1[k] = H2[k]; H2[k] = H3[k]; H3[k] = H4[k];
        }
        const uint32_t boxE = bx_[0] | bx_[2] << 16, boxO = bx_[1] | bx_[3] << 16;
        const uint32_t cE = __byte_perm(cw, 0u, 0x4240), cO = __byte_perm(cw, 0u, 0x4341);
        uint32_t vE = boxE + 25u * (0x00FF00FFu - cE), vO = boxO + 25u * (0x00FF00FFu - cO);
        asm("max.u16x2 %0, %0, %1;" : "+r"(vE) : "r"(0x18E718E7u));   // 6375
        asm("max.u16x2 %0, %0, %1;" : "+r"(vO) : "r"(0x18E718E7u));
        asm("min.u16x2 %0, %0, %1;" : "+r"(vE) : "r"(0x19E619E6u));   // 6630
        asm("min.u16x2 %0, %0, %1;" : "+r"(vO) : "r"(0x19E619E6u));
        vE -= 0x18E718E7u;
        vO -= 0x18E718E7u;
        const uint32_t lapw = vE | vO << 8;          // lanes <= 255: bytes p0, p1, p2, p3
        // Harris (a10) on ext rows r, r+1, r+2 (image rows y-1, y, y+1)
        const HS c = hsum_row(S.fx[r + 2], S.fy[r + 2], G);
        const float2 two = f2(2.f, 2.f);
        const float2 sxxE = add2(fma2(two, b.xxE, a.xxE), c.xxE), sxxO = add2(fma2(two, b.xxO, a.xxO), c.xxO);
        const float2 syyE = add2(fma2(two, b.yyE, a.yyE), c.yyE), syyO = add2(fma2(two, b.yyO, a.yyO), c.yyO);
        const float2 sxyE = add2(fma2(two, b.xyE, a.xyE), c.xyE), sxyO = add2(fma2(two, b.xyO, a.xyO), c.xyO);
        int h0, h1, h2, h3;
        harris2(sxxE, syyE, sxyE, thr_f, thr_err, thr, h0, h2);
        harris2(sxxO, syyO, sxyO, thr_f, thr_err, thr, h1, h3);
        // Sobel magnitude (a9) and the optional dx / dy images, ext row r + 1
        const float4 X = *reinterpret_cast<const float4 *>(&S.fx[r + 1][4 * G]);
        const float4 Y = *reinterpret_cast<const float4 *>(&S.fy[r + 1][4 * G]);
        const float2 nE = fma2(f2(X.x, X.y), f2(X.x, X.y), mul2(f2(Y.x, Y.y), f2(Y.x, Y.y)));
        const float2 nO = fma2(f2(X.z, X.w), f2(X.z, X.w), mul2(f2(Y.z, Y.w), f2(Y.z, Y.w)));
        const uint32_t magw = (uint32_t)mag_f(nE.x) | (uint32_t)mag_f(nO.x) << 8 | (uint32_t)mag_f(nE.y) << 16 |
                              (uint32_t)mag_f(nO.y) << 24;
        const uint32_t harw = (uint32_t)h0 | (uint32_t)h1 << 8 | (uint32_t)h2 << 16 | (uint32_t)h3 << 24;
        if (full) {
            *reinterpret_cast<uint32_t *>(p.lap + off) = lapw;
            *reinterpret_cast<uint32_t *>(p.har + off) = harw;
            *reinterpret_cast<uint32_t *>(p.mag + off) = magw;
            if (p.dx) *reinterpret_cast<uint2 *>(p.dx + off) = make_uint2(pack16((int)X.x, (int)X.z), pack16((int)X.y, (int)X.w));
            if (p.dy) *reinterpret_cast<uint2 *>(p.dy + off) = make_uint2(pack16((int)Y.x, (int)Y.z), pack16((int)Y.y, (int)Y.w));
        } else {   // the image's last, partial 4-pixel group
            const int dxv[4] = {(int)X.x, (int)X.z, (int)X.y, (int)X.w}, dyv[4] = {(int)Y.x, (int)Y.z, (int)Y.y, (int)Y.w};
            for (int k = 0; k < 4 && x + k < p.w; ++k) {
                p.lap[off + k] = (uint8_t)(lapw >> (8 * k));
                p.har[off + k] = (uint8_t)(harw >> (8 * k));
                p.mag[off + k] = (uint8_t)(magw >> (8 * k));
                if (p.dx) p.dx[off + k] = (int16_t)dxv[k];
                if (p.dy) p.dy[off + k] = (int16_t)dyv[k];
            }
        }
        a = b;
        b = c;
    }
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
    const int nbx = (w + TW - 1) / TW, nby = (h + TH - 1) / TH;
    p.nbx = nbx;
    p.nby = nby;
    // Body tiles (Listing 3 at tile granularity: the whole staged window inside the image,
    // 16-B aligned rows, full 4-pixel stores): the fast Body kernel; the frame of border
    // tiles: the general kernel.  ISP_NAIVE / unaligned images: the general kernel alone.
    p.bx0 = 1;
    p.bx1 = std::max(1, std::min(nbx, (w - TW - XO) / TW + 1));
    p.by0 = 1;
    p.by1 = std::max(1, std::min(nby, (h - TH - 2) / TH + 1));
    // one launch of the tile-ISP kernel when the image is at least 2 x 2 tiles + halo (single
    // reflections suffice at its borders); ISP_NAIVE, unaligned or tiny images: the general kernel
    const bool body = !p.naive && p.vec && p.vec_out && p.bx1 > p.bx0 && p.by1 > p.by0 && w >= 2 * TW && h >= 2 * TH &&
                      !getenv("ISP_FUSED_V1");
    // ISP_AUTO / ISP_TMA: the warp-strip band kernel (band_u8.cu) when eligible;
    // ISP_BLOCK / ISP_WARP: the tile-ISP kernel above; ISP_NAIVE: the general kernel
    const bool band = (variant == ISP_AUTO || variant == ISP_TMA) &&
                      ispi_band_fused_ok(img, w, h, pitch, mag, lap, harris, dx, dy, out_pitch);
    cudaError_t e = cudaSuccess;
    if (band) {
        e = ispi_fused_band(img, w, h, pitch, border_mode, const_val, harris_const, thr, dx, dy, mag, lap, harris,
                            out_pitch, (cudaStream_t)stream);
    } else if (body) {
        static bool attr = false;
        if (!attr) {
            cudaFuncSetAttribute(k_fused_body, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(BodySmem));
            attr = true;
        }
        k_fused_body<<<nbx * nby, NT, sizeof(BodySmem), (cudaStream_t)stream>>>(p);
    } else {
        k_fused_cfg3<<<dim3(nbx, nby), NT, 0, (cudaStream_t)stream>>>(p);
    }
    if (e == cudaSuccess) e = cudaGetLastError();
    if (e != cudaSuccess) return ispi_fail(ISP_ECUDA, "isp_pipeline_cfg3_u8: %s", cudaGetErrorString(e));
    return ISP_OK;
}
