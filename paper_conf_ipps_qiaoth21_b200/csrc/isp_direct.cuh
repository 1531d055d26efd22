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
    const int hx = p.mw / 2, hy = p.mh / 2;
    for (int o = 0; o < rows; ++o) {
        const int y = y0 + o;
        typename Op::A acc;
        Op::init(p, acc, x0, y);
        for (int j = 0; j < p.mh; ++j) {
            bool rowok;
            const int yy = map_row<MODE, CK>(y + j - hy, g, rowok);
            const T *__restrict__ row = p.in + (ptrdiff_t)yy * g.in_pitch;
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
    const int bx = blockIdx.x, by = blockIdx.y;
    const int gw = bx * nwarp + warp;
    const int x0 = (gw * 32 + lane) * Op::PX;
    int y0, rows;
    block_rows(p.g, by, gridDim.y, y0, rows);
    if constexpr (DISP == DISP_NAIVE) {
        direct_body<Op, MODE, CK_ALL>(p, x0, y0, rows);
    } else if constexpr (DISP == DISP_NAIVE_GEN) {
        direct_body<Op, MODE, CK_ALL | CK_GEN>(p, x0, y0, rows);
    } else {
        const int rg = region_of(p.g, bx, by, gw, p.g.warp_level != 0);
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

// Generic f32 local operator with a runtime window (<= 31 x 31).  Same FMA order as
// OpConvF32 (row-major taps), so both families give identical bits.
struct DOpConvF32 {
    using Tin = float;
    static constexpr int PX = 4, MAXT = 31 * 31;
    struct Params {
        Geom g;
        const float *in;
        float cval;
        float *out;
        int mw, mh;
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
};

// Generic u8 local operator, runtime window, int32 mask.
struct DOpConvU8 {
    using Tin = uint8_t;
    static constexpr int PX = 4, MAXT = 31 * 31;
    struct Params {
        Geom g;
        const uint8_t *in;
        uint8_t cval;
        uint8_t *out;
        int mw, mh;
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
    struct Params {
        Geom g;
        const float *in;
        float cval;
        float *out;
        int mw, mh;
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
    __device__ __forceinline__ static void tap(const Params &p, int j, int i, const float (&win)[PX], A &a)
    {
        const float ls = p.ls[j * p.mw + i];
#pragma unroll
        for (int e = 0; e < PX; ++e) {
            const float d = win[e] - a.c[e];
            const float wgt = ex2_approx(fmaf(d * d, p.kr, ls));
            a.num[e] = fmaf(wgt, win[e], a.num[e]);
            a.den[e] += wgt;
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
};

}  // namespace ispk
