// tile_u8.cu -- tile-staged ISP kernels for the cfg3 u8 / i16 operators (round 2):
// Laplace 5x5 (a8) and Harris over (dx, dy) (a10), the ISP_TMA variant of
// isp_laplace5_u8 / isp_harris_u8.  Same structure as the fused cfg3 kernel:
//
//   * a CTA owns a 128 x TH output tile; the tile + halo is staged in shared memory --
//     Body tiles (Listing 3 at tile granularity: window inside the image) with unchecked
//     16-byte loads, border tiles row by row through the border pattern (reading A21);
//   * every lane computes 4 adjacent pixels per row and walks TH/4 rows with register
//     rings -- Laplace: horizontal 5-sums by DP4A on byte windows, the clamp on u16x2
//     lanes; Harris: exact integer products / window sums in packed FP32 (< 2^24) and the
//     response in f32 with the rigorous bound of the fused kernel (exact f64 fallback).
//
// The border handling of each operator applies to its own input image, so the
// patterned staging is the whole of it.  Results are the oracle's bit for bit.
#include <cuda_runtime.h>
#include <stdint.h>

#include <algorithm>

#include "../../include/isp.h"
#include "internal.h"
#include "harris_core.cuh"

namespace {

constexpr int NT = 128, TW = 128;
#ifndef TILE_U8_TH
#define TILE_U8_TH 32   // 32 measured best of 16 / 32 / 64 (Laplace 19.5 us, Harris 54.8 us at 4096^2)
#endif
constexpr int TH = TILE_U8_TH, RPW = TH / (NT / 32);

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

struct TileGeom {
    int w, h, pitch, out_pitch, mode, nbx, nby, bx0, bx1, by0, by1;
};

// Tile order: border tiles first (patterned staging is slower), then the Body tiles.
__device__ __forceinline__ void tile_of(const TileGeom &g, int k, int &bx, int &by)
{
    const int iw = g.bx1 - g.bx0, nb_in = iw * (g.by1 - g.by0), nframe = g.nbx * g.nby - nb_in;
    if (k >= nframe) {
        k -= nframe;
        bx = g.bx0 + k % iw;
        by = g.by0 + k / iw;
        return;
    }
    const int per_mid = g.nbx - iw, top = g.by0 * g.nbx, mid = (g.by1 - g.by0) * per_mid;
    if (k < top) { by = k / g.nbx; bx = k % g.nbx; return; }
    k -= top;
    if (k < mid) {
        by = g.by0 + k / per_mid;
        const int j = k % per_mid;
        bx = j < g.bx0 ? j : j + iw;
        return;
    }
    k -= mid;
    by = g.by1 + k / g.nbx;
    bx = k % g.nbx;
}

// Stage rows [y0 - HY, y0 + TH + HY) x columns [x0 - XO, x0 + TW + XO) of an image with
// element type T into s (row stride SW elements).  Body: 16-byte vectors, unchecked.
template <class T, int HY, int XO>
__device__ __forceinline__ void stage(const T *img, const TileGeom &g, T cval, bool body, int x0, int y0, T *s)
{
    constexpr int SW = TW + 2 * XO, SH = TH + 2 * HY, EPV = 16 / (int)sizeof(T), VPR = SW / EPV;
    for (int k = threadIdx.x; k < SH * VPR; k += NT) {
        const int r = k / VPR, c = k % VPR;
        const int y = y0 - HY + r, xs = x0 - XO + c * EPV;
        T *dst = s + r * SW + c * EPV;
        if (body) {
            *reinterpret_cast<uint4 *>(dst) = __ldg(reinterpret_cast<const uint4 *>(img + (size_t)y * g.pitch + xs));
            continue;
        }
        const int yy = bmap1(g.mode, y, g.h);
        if (yy >= 0 && xs >= 0 && xs + EPV <= g.w) {
            *reinterpret_cast<uint4 *>(dst) = __ldg(reinterpret_cast<const uint4 *>(img + (size_t)yy * g.pitch + xs));
        } else {
            for (int e = 0; e < EPV; ++e) {
                const int xx = bmap1(g.mode, xs + e, g.w);
                dst[e] = (yy < 0 || xx < 0) ? cval : img[(size_t)yy * g.pitch + xx];
            }
        }
    }
}

__device__ __forceinline__ uint32_t lw(const uint8_t *p) { return *reinterpret_cast<const uint32_t *>(p); }

// ------------------------------------------------------------------------------ Laplace
struct LapParams {
    TileGeom g;
    const uint8_t *img;
    uint8_t *out;
    uint8_t cval;
};

constexpr int LXO = 16, LSW = TW + 2 * LXO, LSH = TH + 4;

__global__ void __launch_bounds__(NT) k_lap_tile(const __grid_constant__ LapParams p)
{
    __shared__ __align__(16) uint8_t s[LSH * LSW];
    asm volatile("griddepcontrol.wait;" ::: "memory");
    const TileGeom &g = p.g;
    int bx, by;
    tile_of(g, (int)blockIdx.x, bx, by);
    const int x0 = bx * TW, y0 = by * TH;
    const bool body = bx >= g.bx0 && bx < g.bx1 && by >= g.by0 && by < g.by1;
    stage<uint8_t, 2, LXO>(p.img, g, p.cval, body, x0, y0, s);
    __syncthreads();
    const int lane = threadIdx.x & 31, xr = 4 * lane, x = x0 + xr;
    const int rbeg = (threadIdx.x >> 5) * RPW, rend = min(rbeg + RPW, g.h - y0);
    if (rbeg >= rend || x >= g.w) return;
    const uint32_t ones = 0x01010101u;
    auto h5 = [&](int sr, int (&H)[4]) {   // horizontal 5-sums of staged row sr (DP4A)
        const uint8_t *row = s + sr * LSW + LXO + xr;
        const uint32_t L = lw(row - 4), B = lw(row), R = lw(row + 4);
        H[0] = (int)__dp4a(__funnelshift_r(L, B, 16), ones, (B >> 16) & 0xffu);
        H[1] = (int)__dp4a(__funnelshift_r(L, B, 24), ones, B >> 24);
        H[2] = (int)__dp4a(B, ones, R & 0xffu);
        H[3] = (int)__dp4a(__funnelshift_r(B, R, 8), ones, (R >> 8) & 0xffu);
    };
    int H0[4], H1[4], H2[4], H3[4];
    h5(rbeg, H0); h5(rbeg + 1, H1); h5(rbeg + 2, H2); h5(rbeg + 3, H3);
    const bool full = x + 3 < g.w;
#pragma unroll 1
    for (int r = rbeg; r < rend; ++r) {
        int H4[4];
        h5(r + 4, H4);
        uint32_t bx_[4];
#pragma unroll
        for (int k = 0; k < 4; ++k) {
            bx_[k] = (uint32_t)(H0[k] + H1[k] + H2[k] + H3[k] + H4[k]);
            H0[k] = H1[k]; H1[k] = H2[k]; H2[k] = H3[k]; H3[k] = H4[k];
        }
        // clamp(box - 25 c, 0, 255) on u16x2 lanes: v = box + 25 (255 - c) in [0, 12750]
        const uint32_t cw = lw(s + (r + 2) * LSW + LXO + xr);
        const uint32_t cE = __byte_perm(cw, 0u, 0x4240), cO = __byte_perm(cw, 0u, 0x4341);
        uint32_t vE = (bx_[0] | bx_[2] << 16) + 25u * (0x00FF00FFu - cE);
        uint32_t vO = (bx_[1] | bx_[3] << 16) + 25u * (0x00FF00FFu - cO);
        asm("max.u16x2 %0, %0, %1;" : "+r"(vE) : "r"(0x18E718E7u));
        asm("max.u16x2 %0, %0, %1;" : "+r"(vO) : "r"(0x18E718E7u));
        asm("min.u16x2 %0, %0, %1;" : "+r"(vE) : "r"(0x19E619E6u));
        asm("min.u16x2 %0, %0, %1;" : "+r"(vO) : "r"(0x19E619E6u));
        const uint32_t lapw = (vE - 0x18E718E7u) | (vO - 0x18E718E7u) << 8;
        uint8_t *o = p.out + (size_t)(y0 + r) * g.out_pitch + x;
        if (full) {
            *reinterpret_cast<uint32_t *>(o) = lapw;
        } else {
            for (int k = 0; k < 4 && x + k < g.w; ++k) o[k] = (uint8_t)(lapw >> (8 * k));
        }
    }
}

// ------------------------------------------------------------------------------ Harris
struct HarParams {
    TileGeom g;
    const int16_t *dx, *dy;
    uint8_t *out;
    int16_t cval;
    long long thr;
};

constexpr int HXO = 8, HSW = TW + 2 * HXO, HSH = TH + 2;   // int16 elements

struct HS { float2 xxE, xxO, yyE, yyO, xyE, xyO; };

// Horizontal [1,2,1] sums of xx, yy, xy on staged row sr for the lane's 4 pixels, pairs
// E = (p0, p2), O = (p1, p3); products of integers <= 1020 are exact in f32.
__device__ __forceinline__ HS hsum_row(const int16_t *sx, const int16_t *sy, int sr, int xr)
{
    const int16_t *rx = sx + sr * HSW + HXO + xr, *ry = sy + sr * HSW + HXO + xr;
    const uint2 X = *reinterpret_cast<const uint2 *>(rx), Y = *reinterpret_cast<const uint2 *>(ry);
    const float xl = (float)rx[-1], yl = (float)ry[-1], xr4 = (float)rx[4], yr4 = (float)ry[4];
    const float x0 = i2f((int)(int16_t)(X.x & 0xffff)), x1 = i2f((int)X.x >> 16);
    const float x2 = i2f((int)(int16_t)(X.y & 0xffff)), x3 = i2f((int)X.y >> 16);
    const float y0 = i2f((int)(int16_t)(Y.x & 0xffff)), y1 = i2f((int)Y.x >> 16);
    const float y2 = i2f((int)(int16_t)(Y.y & 0xffff)), y3 = i2f((int)Y.y >> 16);
    const float2 xE = f2(x0, x2), xO = f2(x1, x3), yE = f2(y0, y2), yO = f2(y1, y3);
    const float2 xxE = mul2(xE, xE), xxO = mul2(xO, xO), yyE = mul2(yE, yE), yyO = mul2(yO, yO);
    const float2 xyE = mul2(xE, yE), xyO = mul2(xO, yO);
    const float2 xxA = f2(xl * xl, xxO.x), xxB = f2(xxE.y, xr4 * xr4);
    const float2 yyA = f2(yl * yl, yyO.x), yyB = f2(yyE.y, yr4 * yr4);
    const float2 xyA = f2(xl * yl, xyO.x), xyB = f2(xyE.y, xr4 * yr4);
    const float2 two = f2(2.f, 2.f);
    HS h;
    h.xxE = add2(fma2(two, xxE, xxA), xxO);
    h.xxO = add2(fma2(two, xxO, xxE), xxB);
    h.yyE = add2(fma2(two, yyE, yyA), yyO);
    h.yyO = add2(fma2(two, yyO, yyE), yyB);
    h.xyE = add2(fma2(two, xyE, xyA), xyO);
    h.xyO = add2(fma2(two, xyO, xyE), xyB);
    return h;
}

__global__ void __launch_bounds__(NT) k_harris_tile(const __grid_constant__ HarParams p)
{
    __shared__ __align__(16) int16_t sx[HSH * HSW];
    __shared__ __align__(16) int16_t sy[HSH * HSW];
    asm volatile("griddepcontrol.wait;" ::: "memory");
    const TileGeom &g = p.g;
    int bx, by;
    tile_of(g, (int)blockIdx.x, bx, by);
    const int x0 = bx * TW, y0 = by * TH;
    const bool body = bx >= g.bx0 && bx < g.bx1 && by >= g.by0 && by < g.by1;
    stage<int16_t, 1, HXO>(p.dx, g, p.cval, body, x0, y0, sx);
    stage<int16_t, 1, HXO>(p.dy, g, p.cval, body, x0, y0, sy);
    __syncthreads();
    const int lane = threadIdx.x & 31, xr = 4 * lane, x = x0 + xr;
    const int rbeg = (threadIdx.x >> 5) * RPW, rend = min(rbeg + RPW, g.h - y0);
    if (rbeg >= rend || x >= g.w) return;
    const double thr = (double)max(-9007199254740992ll, min(9007199254740992ll, p.thr));
    const float thr_f = (float)thr;
    const float thr_err = thr_bound(thr_f);
    HS a = hsum_row(sx, sy, rbeg, xr), b = hsum_row(sx, sy, rbeg + 1, xr);
    const bool full = x + 3 < g.w;
    const float2 two = f2(2.f, 2.f);
#pragma unroll 1
    for (int r = rbeg; r < rend; ++r) {
        const HS c = hsum_row(sx, sy, r + 2, xr);
        const float2 sxxE = add2(fma2(two, b.xxE, a.xxE), c.xxE), sxxO = add2(fma2(two, b.xxO, a.xxO), c.xxO);
        const float2 syyE = add2(fma2(two, b.yyE, a.yyE), c.yyE), syyO = add2(fma2(two, b.yyO, a.yyO), c.yyO);
        const float2 sxyE = add2(fma2(two, b.xyE, a.xyE), c.xyE), sxyO = add2(fma2(two, b.xyO, a.xyO), c.xyO);
        int h0, h1, h2, h3;
        harris2(sxxE, syyE, sxyE, thr_f, thr_err, thr, h0, h2);
        harris2(sxxO, syyO, sxyO, thr_f, thr_err, thr, h1, h3);
        const uint32_t w4 = (uint32_t)h0 | (uint32_t)h1 << 8 | (uint32_t)h2 << 16 | (uint32_t)h3 << 24;
        uint8_t *o = p.out + (size_t)(y0 + r) * g.out_pitch + x;
        if (full) {
            *reinterpret_cast<uint32_t *>(o) = w4;
        } else {
            for (int k = 0; k < 4 && x + k < g.w; ++k) o[k] = (uint8_t)(w4 >> (8 * k));
        }
        a = b;
        b = c;
    }
}

// Body rectangle of the tile grid: tiles whose staged window [x0 - XO, x0 + TW + XO) x
// [y0 - HY, y0 + TH + HY) is inside the image.
TileGeom tile_geom(int w, int h, int pitch, int out_pitch, int mode, int xo, int hy)
{
    TileGeom g{};
    g.w = w; g.h = h; g.pitch = pitch; g.out_pitch = out_pitch; g.mode = mode;
    g.nbx = (w + TW - 1) / TW;
    g.nby = (h + TH - 1) / TH;
    g.bx0 = (xo + TW - 1) / TW;
    g.bx1 = std::max(g.bx0, std::min(g.nbx, (w - TW - xo) / TW + 1));
    g.by0 = (hy + TH - 1) / TH;
    g.by1 = std::max(g.by0, std::min(g.nby, (h - TH - hy) / TH + 1));
    return g;
}

cudaError_t launch_tile(const void *fn, void *params, int nblocks, cudaStream_t st)
{
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3(nblocks);
    cfg.blockDim = dim3(NT);
    cfg.stream = st;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    void *args[] = {params};
    return cudaLaunchKernelExC(&cfg, fn, args);
}

}  // namespace

// Eligibility of the tile kernels: 16-B aligned rows (the Body tiles' vector loads), 4-B
// aligned outputs, and at least 2 x 2 tiles so border overshoots need one reflection.
bool ispi_tile_ok(const void *in0, const void *in1, int elem, int w, int h, int pitch, const void *out,
                  int out_pitch)
{
    auto al = [](const void *q, long long pb, int v) { return q && ((uintptr_t)q % v) == 0 && (pb % v) == 0; };
    return al(in0, (long long)pitch * elem, 16) && (!in1 || al(in1, (long long)pitch * elem, 16)) &&
           al(out, out_pitch, 4) && w >= 2 * TW + 32 && h >= 2 * TH + 4;
}

void ispi_tile_shape(int *tw, int *th) { *tw = TW; *th = TH; }

cudaError_t ispi_laplace_tile(const uint8_t *img, int w, int h, int pitch, int mode, int cval, uint8_t *out,
                              int out_pitch, cudaStream_t st, int bounds[4])
{
    LapParams p{};
    p.g = tile_geom(w, h, pitch, out_pitch, mode, LXO, 2);
    p.img = img;
    p.out = out;
    p.cval = (uint8_t)cval;
    bounds[0] = p.g.bx0; bounds[1] = p.g.bx1; bounds[2] = p.g.by0; bounds[3] = p.g.by1;
    return launch_tile((const void *)k_lap_tile, &p, p.g.nbx * p.g.nby, st);
}

cudaError_t ispi_harris_tile(const int16_t *dx, const int16_t *dy, int w, int h, int pitch, int mode, int cval,
                             long long thr, uint8_t *out, int out_pitch, cudaStream_t st, int bounds[4])
{
    HarParams p{};
    p.g = tile_geom(w, h, pitch, out_pitch, mode, HXO, 1);
    p.dx = dx;
    p.dy = dy;
    p.out = out;
    p.cval = (int16_t)cval;
    p.thr = thr;
    bounds[0] = p.g.bx0; bounds[1] = p.g.bx1; bounds[2] = p.g.by0; bounds[3] = p.g.by1;
    return launch_tile((const void *)k_harris_tile, &p, p.g.nbx * p.g.nby, st);
}

// Resident CTAs per SM of the tile kernels (occupancy term O of Eq. 10).
int ispi_tile_blocks_per_sm(int which)
{
    int nb = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, which == 0 ? (const void *)k_lap_tile
                                                                      : (const void *)k_harris_tile, NT, 0) !=
        cudaSuccess) {
        cudaGetLastError();
        return 0;
    }
    return nb;
}
