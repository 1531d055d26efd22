// isp_direct.cuh -- runtime-window ("direct") family of region-specialised kernels.
//
// Used for windows that are not compiled into the streaming engine (any odd m x n up
// to 31 x 31) and for the Bilateral filter, the paper's motivating
// example.  Structure follows the paper's per-tap address calculation: for
// every window row j the row index is mapped (T/B regions only), and every loaded
// column is mapped (L/R regions only); Body runs no checks.  Each thread produces PX
// horizontally adjacent outputs and keeps a PX-wide shift register of the current
// window column, so one load serves PX taps.
#pragma once
#include "isp_ops.cuh"
#include "kernels.h"

namespace ispk {

template <class T, int MODE, int CK>
__device__ __forceinline__ T load_x(const T *__restrict__ row, bool rowok, int x, const Geom &g, T cval)
{
    constexpr bool GEN = (CK & CK_GEN) != 0;
    if constexpr (MODE == CONSTANT) {
        bool ok = rowok && inbounds<(CK & CK_L) != 0, (CK & CK_R) != 0>(x, g.w);
        return ok ? __ldg(row + x) : cval;
    } else {
        x = bmap<MODE, (CK & CK_L) != 0, (CK & CK_R) != 0, GEN>(x, g.w);
        return __ldg(row + x);
    }
}

template <class Op, int MODE, int CK>
__device__ __forceinline__ void direct_body(const typename Op::Params &p, int x0, int y0, int rows)
{
    using T = typename Op::Tin;
    constexpr int PX = Op::PX;
    const Geom &g = p.g;
    // anchor (ax, ay): taps at offsets (i - ax, j - ay); the centre for dense windows,
    // anywhere for cropped sparse masks (reading A31)
    const int hx = p.ax, hy = p.ay;
    for (int o = 0; o < rows; ++o) {
        const int y = y0 + o;
        typename Op::A acc;
        Op::init(p, acc, x0, y);
        for (int j = 0; j < p.mh; ++j) {
            bool rowok;
            const int yy = map_row<MODE, CK>(y + j - hy, g, rowok);
            const T *__restrict__ row = row_base<CK>(p.in, yy, g);
            T win[PX];
#pragma unroll
            for (int e = 0; e < PX; ++e) win[e] = load_x<T, MODE, CK>(row, rowok, x0 - hx + e, g, p.cval);
            Op::tap(p, j, 0, win, acc);
            for (int i = 1; i < p.mw; ++i) {
#pragma unroll
                for (int e = 0; e < PX - 1; ++e) win[e] = win[e + 1];
                win[PX - 1] = load_x<T, MODE, CK>(row, rowok, x0 - hx + i + PX - 1, g, p.cval);
                Op::tap(p, j, i, win, acc);
            }
        }
        Op::template store<CK>(p, acc, x0, y);
    }
}

template <class Op, int MODE, int DISP>
__global__ void __launch_bounds__(256) k_direct(const __grid_constant__ typename Op::Params p)
{
    pdl_launch_dependents();
    pdl_wait();
    const int lane = threadIdx.x & 31;
    const int warp = threadIdx.x >> 5;
    const int nwarp = blockDim.x >> 5;
    // split launches (variant ISP_SPLIT, one kernel per region, P:L90 ablation): the
    // launch covers one region's block rectangle starting at (bx0, by0)
    const int bx = blockIdx.x + p.g.bx0, by = blockIdx.y + p.g.by0;
    const int gw = bx * nwarp + warp;
    const int x0 = (gw * 32 + lane) * Op::PX;
    int y0, rows;
    block_rows(p.g, by, gridDim.y, y0, rows);
    if constexpr (DISP == DISP_NAIVE) {
        direct_body<Op, MODE, CK_ALL>(p, x0, y0, rows);
    } else if constexpr (DISP == DISP_NAIVE_GEN) {
        direct_body<Op, MODE, CK_ALL | CK_GEN>(p, x0, y0, rows);
    } else {
        const int rg = p.g.force_rg >= 0 ? p.g.force_rg : region_of(p.g, bx, by, gw, p.g.warp_level != 0);
        switch (rg) {
        case RG_TL: direct_body<Op, MODE, region_checks(RG_TL)>(p, x0, y0, rows); break;
        case RG_TR: direct_body<Op, MODE, region_checks(RG_TR)>(p, x0, y0, rows); break;
        case RG_T: direct_body<Op, MODE, region_checks(RG_T)>(p, x0, y0, rows); break;
        case RG_BL: direct_body<Op, MODE, region_checks(RG_BL)>(p, x0, y0, rows); break;
        case RG_BR: direct_body<Op, MODE, region_checks(RG_BR)>(p, x0, y0, rows); break;
        case RG_B: direct_body<Op, MODE, region_checks(RG_B)>(p, x0, y0, rows); break;
        case RG_R: direct_body<Op, MODE, region_checks(RG_R)>(p, x0, y0, rows); break;
        case RG_L: direct_body<Op, MODE, region_checks(RG_L)>(p, x0, y0, rows); break;
        default: direct_body<Op, MODE, 0>(p, x0, y0, rows); break;
        }
    }
}

// ---------------------------------------------------------------------------------
// Shared-memory tiled form of the direct family (variant ISP_TMA for runtime-window ops:
// the staged family of the expensive kernels).  CTA = kTileWarps warps over a tile of
// kTileW x kTileH outputs; each thread owns PX outputs of one row at a stride of 32
// columns, so a tap reads PX conflict-free words of one smem row and no value is moved
// between taps.  ISP lives in the fill (reading A21): the CTA's region (Listing 3 on
// the tile grid, Eq. 2 with this tile shape) decides which sides of the (tile + halo)
// fill go through the border pattern; a Body CTA copies unchecked.  The compute loop
// has no checks in any region and runs the same per-output operations in the same
// order as direct_body, so all variants give identical bits.
// ---------------------------------------------------------------------------------
constexpr int kTileWarps = TILE_THREADS / 32, kTileThreads = TILE_THREADS, kTileH = TILE_H;

template <class Op, int MODE, int CK>
__device__ __forceinline__ void tile_fill(const typename Op::Params &p, typename Op::Tin *tile, int X0, int Y0,
                                          int SW, int SH)
{
    using T = typename Op::Tin;
    const Geom &g = p.g;
    const int hx = p.ax, hy = p.ay;
    for (int r = threadIdx.x / 32; r < SH; r += kTileWarps) {
        bool rowok;
        const int yy = map_row<MODE, CK>(Y0 - hy + r, g, rowok);
        const T *__restrict__ row = row_base<CK>(p.in, yy, g);
        T *dst = tile + r * SW;
        for (int c = threadIdx.x & 31; c < SW; c += 32) {
            const int x = X0 - hx + c;
            if constexpr ((CK & (CK_L | CK_R | CK_T | CK_B)) == 0) {
                dst[c] = __ldg(row + x);                       // Body: no checks
            } else {
                dst[c] = load_x<T, MODE, CK>(row, rowok, x, g, p.cval);
            }
        }
    }
}

template <class Op, int MODE, int CK>
__device__ __forceinline__ void tile_body(const typename Op::Params &p, typename Op::Tin *tile)
{
    using T = typename Op::Tin;
    constexpr int PX = Op::PX, TW = 32 * PX;
    static_assert(PX == TILE_PX, "the planner sizes tiles with TILE_PX");
    const int X0 = blockIdx.x * TW, Y0 = p.g.oy0 + blockIdx.y * kTileH;
    const int SW = TW + p.mw - 1, SH = kTileH + p.mh - 1;
    tile_fill<Op, MODE, CK>(p, tile, X0, Y0, SW, SH);
    __syncthreads();
    const int lane = threadIdx.x & 31;
    for (int o = threadIdx.x / 32; o < kTileH; o += kTileWarps) {
        const int y = Y0 + o;
        if ((CK & CK_B) && y >= p.g.y_end) break;
        typename Op::A acc;
        Op::init_tile(p, acc, tile + (o + p.ay) * SW + p.ax + lane);
        for (int j = 0; j < p.mh; ++j) {
            const T *srow = tile + (o + j) * SW + lane;
#pragma unroll 2
            for (int i = 0; i < p.mw; ++i) {
                T win[PX];
#pragma unroll
                for (int e = 0; e < PX; ++e) win[e] = srow[i + 32 * e];
                Op::tap(p, j, i, win, acc);
            }
        }
        Op::template store_strided<CK>(p, acc, X0 + lane, y);
    }
}

template <class Op, int MODE>
__global__ void __launch_bounds__(kTileThreads) k_tile(const __grid_constant__ typename Op::Params p)
{
    extern __shared__ __align__(16) unsigned char tile_smem[];
    auto *tile = reinterpret_cast<typename Op::Tin *>(tile_smem);
    pdl_launch_dependents();
    pdl_wait();
    switch (region_of(p.g, blockIdx.x, blockIdx.y, 0, false)) {
    case RG_TL: tile_body<Op, MODE, region_checks(RG_TL)>(p, tile); break;
    case RG_TR: tile_body<Op, MODE, region_checks(RG_TR)>(p, tile); break;
    case RG_T: tile_body<Op, MODE, region_checks(RG_T)>(p, tile); break;
    case RG_BL: tile_body<Op, MODE, region_checks(RG_BL)>(p, tile); break;
    case RG_BR: tile_body<Op, MODE, region_checks(RG_BR)>(p, tile); break;
    case RG_B: tile_body<Op, MODE, region_checks(RG_B)>(p, tile); break;
    case RG_R: tile_body<Op, MODE, region_checks(RG_R)>(p, tile); break;
    case RG_L: tile_body<Op, MODE, region_checks(RG_L)>(p, tile); break;
    default: tile_body<Op, MODE, 0>(p, tile); break;
    }
}

// Strided store of the tiled form: element e is column x + 32 e (guarded in R regions).
template <int CK, class T, int PX>
__device__ __forceinline__ void store_strided_px(T *__restrict__ row, int x, int w, const T (&v)[PX])
{
#pragma unroll
    for (int e = 0; e < PX; ++e)
        if (!(CK & CK_R) || x + 32 * e < w) row[x + 32 * e] = v[e];
}

// Generic f32 local operator with a runtime window (<= 31 x 31).  Same FMA order as
// OpConvF32 (row-major taps), so both families give identical bits.
struct DOpConvF32 {
    using Tin = float;
    static constexpr int PX = 4, MAXT = 31 * 31;
    static constexpr bool TILED = true;
    struct Params {
        Geom g;
        const float *in;
        float cval;
        float *out;
        int mw, mh;
        int ax, ay;   // anchor: tap (i, j) reads offset (i - ax, j - ay)
        float mask[MAXT];
    };
    struct A { float v[PX]; };
    __device__ __forceinline__ static void init(const Params &, A &a, int, int)
    {
#pragma unroll
        for (int e = 0; e < PX; ++e) a.v[e] = 0.f;
    }
    __device__ __forceinline__ static void tap(const Params &p, int j, int i, const float (&win)[PX], A &a)
    {
        const float m = p.mask[j * p.mw + i];
#pragma unroll
        for (int e = 0; e < PX; ++e) a.v[e] = fmaf(m, win[e], a.v[e]);
    }
    template <int CK>
    __device__ __forceinline__ static void store(const Params &p, const A &a, int x0, int y)
    {
        store_px<CK, float, PX>(p.out + (ptrdiff_t)(y - p.g.oy0) * p.g.out_pitch, x0, p.g.w, p.g.vec_out, a.v);
    }
    __device__ __forceinline__ static void init_tile(const Params &p, A &a, const float *) { init(p, a, 0, 0); }
    template <int CK>
    __device__ __forceinline__ static void store_strided(const Params &p, const A &a, int x, int y)
    {
        store_strided_px<CK, float, PX>(p.out + (ptrdiff_t)(y - p.g.oy0) * p.g.out_pitch, x, p.g.w, a.v);
    }
};

// Generic u8 local operator, runtime window, int32 mask.
struct DOpConvU8 {
    using Tin = uint8_t;
    static constexpr int PX = 4, MAXT = 31 * 31;
    static constexpr bool TILED = false;
    struct Params {
        Geom g;
        const uint8_t *in;
        uint8_t cval;
        uint8_t *out;
        int mw, mh;
        int ax, ay;   // anchor: tap (i, j) reads offset (i - ax, j - ay)
        U8Round rnd;
        int mask[MAXT];
    };
    struct A { int v[PX]; };
    __device__ __forceinline__ static void init(const Params &, A &a, int, int)
    {
#pragma unroll
        for (int e = 0; e < PX; ++e) a.v[e] = 0;
    }
    __device__ __forceinline__ static void tap(const Params &p, int j, int i, const uint8_t (&win)[PX], A &a)
    {
        const int m = p.mask[j * p.mw + i];
#pragma unroll
        for (int e = 0; e < PX; ++e) a.v[e] += m * (int)win[e];
    }
    template <int CK>
    __device__ __forceinline__ static void store(const Params &p, const A &a, int x0, int y)
    {
        uint8_t o[PX];
#pragma unroll
        for (int e = 0; e < PX; ++e) o[e] = sat_u8(p.rnd(a.v[e]));
        store_px<CK, uint8_t, PX>(p.out + (ptrdiff_t)(y - p.g.oy0) * p.g.out_pitch, x0, p.g.w, p.g.vec_out, o);
    }
};

__device__ __forceinline__ float ex2_approx(float x)
{
    float y;
    asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
    return y;
}

// Bilateral (a11): weight(q) = s(q-p) * r(I_q - I_p) with
// r = exp(-d^2 / (2 sigma_r^2)) = 2^(d^2 * kr), kr = -log2(e) / (2 sigma_r^2), and the
// spatial factor folded into the exponent: weight = 2^(d^2 kr + log2 s(q-p)).
struct DOpBilateral {
    using Tin = float;
    static constexpr int PX = 4, MAXT = 31 * 31;
    static constexpr bool TILED = true;
    struct Params {
        Geom g;
        const float *in;
        float cval;
        float *out;
        int mw, mh;
        int ax, ay;   // anchor: tap (i, j) reads offset (i - ax, j - ay)
        float kr;
        float ls[MAXT];  // log2 of the spatial weights s(dx, dy)
    };
    struct A { float c[PX], num[PX], den[PX]; };
    __device__ __forceinline__ static void init(const Params &p, A &a, int x0, int y)
    {
        const float *row = p.in + (ptrdiff_t)y * p.g.in_pitch;
#pragma unroll
        for (int e = 0; e < PX; ++e) {
            a.c[e] = __ldg(row + min(x0 + e, p.g.w - 1));  // the centre is always inside
            a.num[e] = 0.f;
            a.den[e] = 0.f;
        }
    }
    // per output: d = I_q - I_p, w = 2^(d*d*kr + ls), num += w I_q, den += w -- two outputs
    // per instruction with the sm_100 packed FP32 ops (each lane an IEEE op: the same
    // bits as the scalar sequence)
    __device__ __forceinline__ static void tap(const Params &p, int j, int i, const float (&win)[PX], A &a)
    {
        const float ls = p.ls[j * p.mw + i];
        unsigned long long kr2, ls2;
        asm("mov.b64 %0, {%1, %1};" : "=l"(kr2) : "f"(p.kr));
        asm("mov.b64 %0, {%1, %1};" : "=l"(ls2) : "f"(ls));
#pragma unroll
        for (int e = 0; e < PX; e += 2) {
            unsigned long long wv, nc, d, t, num, den, wg;
            asm("mov.b64 %0, {%1, %2};" : "=l"(wv) : "f"(win[e]), "f"(win[e + 1]));
            asm("mov.b64 %0, {%1, %2};" : "=l"(nc) : "f"(-a.c[e]), "f"(-a.c[e + 1]));
            asm("add.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(wv), "l"(nc));
            asm("mul.rn.f32x2 %0, %1, %1;" : "=l"(t) : "l"(d));
            asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(t) : "l"(t), "l"(kr2), "l"(ls2));
            float t0, t1;
            asm("mov.b64 {%0, %1}, %2;" : "=f"(t0), "=f"(t1) : "l"(t));
            const float w0 = ex2_approx(t0), w1 = ex2_approx(t1);
            asm("mov.b64 %0, {%1, %2};" : "=l"(wg) : "f"(w0), "f"(w1));
            asm("mov.b64 %0, {%1, %2};" : "=l"(num) : "f"(a.num[e]), "f"(a.num[e + 1]));
            asm("mov.b64 %0, {%1, %2};" : "=l"(den) : "f"(a.den[e]), "f"(a.den[e + 1]));
            asm("fma.rn.f32x2 %0, %1, %2, %0;" : "+l"(num) : "l"(wg), "l"(wv));
            asm("add.rn.f32x2 %0, %0, %1;" : "+l"(den) : "l"(wg));
            asm("mov.b64 {%0, %1}, %2;" : "=f"(a.num[e]), "=f"(a.num[e + 1]) : "l"(num));
            asm("mov.b64 {%0, %1}, %2;" : "=f"(a.den[e]), "=f"(a.den[e + 1]) : "l"(den));
        }
    }
    template <int CK>
    __device__ __forceinline__ static void store(const Params &p, const A &a, int x0, int y)
    {
        float o[PX];
#pragma unroll
        for (int e = 0; e < PX; ++e) o[e] = a.num[e] / a.den[e];
        store_px<CK, float, PX>(p.out + (ptrdiff_t)(y - p.g.oy0) * p.g.out_pitch, x0, p.g.w, p.g.vec_out, o);
    }
    // tiled form: centre values from the smem tile (element e at column +32 e)
    __device__ __forceinline__ static void init_tile(const Params &, A &a, const float *ctr)
    {
#pragma unroll
        for (int e = 0; e < PX; ++e) {
            a.c[e] = ctr[32 * e];
            a.num[e] = 0.f;
            a.den[e] = 0.f;
        }
    }
    template <int CK>
    __device__ __forceinline__ static void store_strided(const Params &p, const A &a, int x, int y)
    {
        float o[PX];
#pragma unroll
        for (int e = 0; e < PX; ++e) o[e] = a.num[e] / a.den[e];
        store_strided_px<CK, float, PX>(p.out + (ptrdiff_t)(y - p.g.oy0) * p.g.out_pitch, x, p.g.w, o);
    }
};

}  // namespace ispk
