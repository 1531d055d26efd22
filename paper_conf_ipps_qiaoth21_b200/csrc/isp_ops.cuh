// isp_ops.cuh -- the local operators of the paper's evaluation as streaming
// ops for the region-specialised engine (isp_core.cuh).
//
// Each op decomposes its window into a per-input-row horizontal part (hrow) and a
// vertical accumulation into output-row accumulators (vacc, j = window row), which
// is exact for integer ops and keeps the f32 generic op's row-major FMA order.
#pragma once
#include "isp_core.cuh"

namespace ispk {

template <int PX> struct AccF { float v[PX]; };

// Packed FP32 FMA (sm_100 FFMA2): (a0, a1) = fma(c, (b0, b1), (a0, a1)) -- two IEEE fmaf
// per instruction, bitwise identical to the scalar form; c is broadcast.
__device__ __forceinline__ void fma2(float &a0, float &a1, float c, float b0, float b1)
{
    unsigned long long aa, bb, cc;
    asm("mov.b64 %0, {%1, %2};" : "=l"(aa) : "f"(a0), "f"(a1));
    asm("mov.b64 %0, {%1, %2};" : "=l"(bb) : "f"(b0), "f"(b1));
    asm("mov.b64 %0, {%1, %1};" : "=l"(cc) : "f"(c));
    asm("fma.rn.f32x2 %0, %1, %2, %0;" : "+l"(aa) : "l"(cc), "l"(bb));
    asm("mov.b64 {%0, %1}, %2;" : "=f"(a0), "=f"(a1) : "l"(aa));
}
__device__ __forceinline__ void mul2(float &a0, float &a1, float c, float b0, float b1)
{
    unsigned long long aa, bb, cc;
    asm("mov.b64 %0, {%1, %2};" : "=l"(bb) : "f"(b0), "f"(b1));
    asm("mov.b64 %0, {%1, %1};" : "=l"(cc) : "f"(c));
    asm("mul.rn.f32x2 %0, %1, %2;" : "=l"(aa) : "l"(cc), "l"(bb));
    asm("mov.b64 {%0, %1}, %2;" : "=f"(a0), "=f"(a1) : "l"(aa));
}
template <int PX, int NC> struct AccI { int v[NC][PX]; };

// ---------------------------------------------------------------------------------
// Generic f32 local operator, compile-time MW x MH ("Mask").
// out = sum_j sum_i mask[j][i] * in(x+i-hx, y+j-hy): one FMA chain per output in
// row-major tap order (j outer, i inner) -- identical in every region / variant.
// ---------------------------------------------------------------------------------
template <int MW_, int MH_>
struct OpConvF32 {
    using Tin = float;
    static constexpr int NIN = 1, PX = 4, HX = MW_ / 2, HY = MH_ / 2, MH = MH_, SEGW = PX + 2 * HX;
    static constexpr int PFMAX = 0;
    static constexpr bool ROW_DIRECT = false;
    static constexpr bool SHFL_HALO = false;  // shuffle halo measured slower
    struct Params {
        Geom g;
        const float *in[1];
        float cval;
        float *out;
        float mask[MW_ * MH_];
    };
    struct H { float s[SEGW]; };
    using A = AccF<PX>;
    __host__ __device__ static constexpr bool col_used(int) { return true; }
    __host__ __device__ static constexpr bool row_used(int) { return true; }
    __device__ __forceinline__ static void zero(A &a)
    {
#pragma unroll
        for (int e = 0; e < PX; ++e) a.v[e] = 0.f;
    }
    __device__ __forceinline__ static void hrow(const Params &, const float (&seg)[1][SEGW], H &h)
    {
#pragma unroll
        for (int k = 0; k < SEGW; ++k) h.s[k] = seg[0][k];
    }
    // FIRST: the output row's first tap (j == 0) initialises the accumulator
    template <bool FIRST>
    __device__ __forceinline__ static void vacc(const Params &p, int j, const H &h, A &a)
    {
        // scalar FFMA: the packed form (fma2) makes ptxas take ~20 min on the 7x7 instance
#pragma unroll
        for (int i = 0; i < MW_; ++i)
#pragma unroll
            for (int e = 0; e < PX; ++e)
                a.v[e] = (FIRST && i == 0) ? p.mask[j * MW_] * h.s[e] : fmaf(p.mask[j * MW_ + i], h.s[e + i], a.v[e]);
    }
    template <int CK>
    __device__ __forceinline__ static void store(const Params &p, const A &a, int x0, int y)
    {
        store_px<CK, float, PX>(p.out + (ptrdiff_t)(y - p.g.oy0) * p.g.out_pitch, x0, p.g.w, p.g.vec_out, a.v);
    }
};

// ---------------------------------------------------------------------------------
// Separable f32 operator: row pass then column pass fused per strip (no intermediate
// image).  h = sum_i row[i] in(x+i-hx, .) ; out = sum_j col[j] h(., y+j-hy).
// ---------------------------------------------------------------------------------
template <int MW_, int MH_>
struct OpSepF32 {
    using Tin = float;
    static constexpr int NIN = 1, PX = 4, HX = MW_ / 2, HY = MH_ / 2, MH = MH_, SEGW = PX + 2 * HX;
    static constexpr int PFMAX = 0;
    static constexpr bool ROW_DIRECT = false;
    static constexpr bool SHFL_HALO = false;  // shuffle halo measured slower
    struct Params {
        Geom g;
        const float *in[1];
        float cval;
        float *out;
        float row[MW_];
        float col[MH_];
    };
    struct H { float v[PX]; };
    using A = AccF<PX>;
    __host__ __device__ static constexpr bool col_used(int) { return true; }
    __host__ __device__ static constexpr bool row_used(int) { return true; }
    __device__ __forceinline__ static void zero(A &a)
    {
#pragma unroll
        for (int e = 0; e < PX; ++e) a.v[e] = 0.f;
    }
    __device__ __forceinline__ static void hrow(const Params &p, const float (&seg)[1][SEGW], H &h)
    {
#pragma unroll
        for (int e = 0; e < PX; e += 2) {
            float t0, t1;
            mul2(t0, t1, p.row[0], seg[0][e], seg[0][e + 1]);
#pragma unroll
            for (int i = 1; i < MW_; ++i) fma2(t0, t1, p.row[i], seg[0][e + i], seg[0][e + i + 1]);
            h.v[e] = t0;
            h.v[e + 1] = t1;
        }
    }
    template <bool FIRST>
    __device__ __forceinline__ static void vacc(const Params &p, int j, const H &h, A &a)
    {
#pragma unroll
        for (int e = 0; e < PX; e += 2) {
            if (FIRST) mul2(a.v[e], a.v[e + 1], p.col[j], h.v[e], h.v[e + 1]);
            else fma2(a.v[e], a.v[e + 1], p.col[j], h.v[e], h.v[e + 1]);
        }
    }
    template <int CK>
    __device__ __forceinline__ static void store(const Params &p, const A &a, int x0, int y)
    {
        store_px<CK, float, PX>(p.out + (ptrdiff_t)(y - p.g.oy0) * p.g.out_pitch, x0, p.g.w, p.g.vec_out, a.v);
    }
};

// ---------------------------------------------------------------------------------
// u8 helpers: round-half-up division and saturation (reading A12).
// ---------------------------------------------------------------------------------
struct U8Round {
    int divisor, shift, half; // shift >= 0: divisor == 1 << shift, half = divisor >> 1
    __device__ __forceinline__ int operator()(int acc) const
    {
        if (shift >= 0) return (acc + half) >> shift;            // floor((acc + d/2) / d)
        const int num = 2 * acc + divisor, den = 2 * divisor;     // floor((2acc + d) / (2d))
        int q = num / den;
        if ((num % den != 0) && (num < 0)) q -= 1;
        return q;
    }
};

__device__ __forceinline__ uint8_t sat_u8(int v) { return (uint8_t)min(255, max(0, v)); }

// Generic u8 local operator with an int32 mask, compile-time MW x MH.
template <int MW_, int MH_>
struct OpConvU8 {
    using Tin = uint8_t;
    static constexpr int NIN = 1, PX = kPxU8, HX = MW_ / 2, HY = MH_ / 2, MH = MH_, SEGW = PX + 2 * HX;
    static constexpr int PFMAX = kPfSub;  // rows loaded ahead (latency hiding)
    static constexpr bool ROW_DIRECT = false;
    static constexpr bool SHFL_HALO = false;  // shuffle halo measured slower
    struct Params {
        Geom g;
        const uint8_t *in[1];
        uint8_t cval;
        uint8_t *out;
        U8Round rnd;
        int mask[MW_ * MH_];
    };
    struct H { int s[SEGW]; };
    using A = AccI<PX, 1>;
    __host__ __device__ static constexpr bool col_used(int) { return true; }
    __host__ __device__ static constexpr bool row_used(int) { return true; }
    __device__ __forceinline__ static void zero(A &a)
    {
#pragma unroll
        for (int e = 0; e < PX; ++e) a.v[0][e] = 0;
    }
    __device__ __forceinline__ static void hrow(const Params &, const uint8_t (&seg)[1][SEGW], H &h)
    {
#pragma unroll
        for (int k = 0; k < SEGW; ++k) h.s[k] = seg[0][k];
    }
    template <bool FIRST>
    __device__ __forceinline__ static void vacc(const Params &p, int j, const H &h, A &a)
    {
#pragma unroll
        for (int i = 0; i < MW_; ++i)
#pragma unroll
            for (int e = 0; e < PX; ++e)
                a.v[0][e] = ((FIRST && i == 0) ? 0 : a.v[0][e]) + p.mask[j * MW_ + i] * h.s[e + i];
    }
    template <int CK>
    __device__ __forceinline__ static void store(const Params &p, const A &a, int x0, int y)
    {
        uint8_t o[PX];
#pragma unroll
        for (int e = 0; e < PX; ++e) o[e] = sat_u8(p.rnd(a.v[0][e]));
        store_px<CK, uint8_t, PX>(p.out + (ptrdiff_t)(y - p.g.oy0) * p.g.out_pitch, x0, p.g.w, p.g.vec_out, o);
    }
};

// Separable u8 operator with integer row/col weights (exact: integer intermediates).
template <int MW_, int MH_>
struct OpSepU8 {
    using Tin = uint8_t;
    static constexpr int NIN = 1, PX = kPxU8, HX = MW_ / 2, HY = MH_ / 2, MH = MH_, SEGW = PX + 2 * HX;
    static constexpr int PFMAX = kPfSub;  // rows loaded ahead (latency hiding)
    static constexpr bool ROW_DIRECT = false;
    static constexpr bool SHFL_HALO = false;  // shuffle halo measured slower
    struct Params {
        Geom g;
        const uint8_t *in[1];
        uint8_t cval;
        uint8_t *out;
        U8Round rnd;
        int row[MW_];
        int col[MH_];
    };
    struct H { int v[PX]; };
    using A = AccI<PX, 1>;
    __host__ __device__ static constexpr bool col_used(int) { return true; }
    __host__ __device__ static constexpr bool row_used(int) { return true; }
    __device__ __forceinline__ static void zero(A &a)
    {
#pragma unroll
        for (int e = 0; e < PX; ++e) a.v[0][e] = 0;
    }
    __device__ __forceinline__ static void hrow(const Params &p, const uint8_t (&seg)[1][SEGW], H &h)
    {
#pragma unroll
        for (int e = 0; e < PX; ++e) {
            int t = 0;
#pragma unroll
            for (int i = 0; i < MW_; ++i) t += p.row[i] * (int)seg[0][e + i];
            h.v[e] = t;
        }
    }
    template <bool FIRST>
    __device__ __forceinline__ static void vacc(const Params &p, int j, const H &h, A &a)
    {
#pragma unroll
        for (int e = 0; e < PX; ++e) a.v[0][e] = (FIRST ? 0 : a.v[0][e]) + p.col[j] * h.v[e];
    }
    template <int CK>
    __device__ __forceinline__ static void store(const Params &p, const A &a, int x0, int y)
    {
        uint8_t o[PX];
#pragma unroll
        for (int e = 0; e < PX; ++e) o[e] = sat_u8(p.rnd(a.v[0][e]));
        store_px<CK, uint8_t, PX>(p.out + (ptrdiff_t)(y - p.g.oy0) * p.g.out_pitch, x0, p.g.w, p.g.vec_out, o);
    }
};

// Sobel magnitude min(255, round_half_up(sqrt(n))) for integer n >= 0 (a9), exact:
// for n <= 65280 (= 255.5^2 - 0.25, beyond which the result saturates to 255) sqrt(n)
// stays >= 1.5e-3 from every integer - 1/2 (n and k^2 +- k are integers), while
// sqrt.approx.f32 errs by a few ulp (< 1e-4 at 255.5), so floor(sqrt(n) + 1/2) taken in
// f32 is the exact rounding.
__device__ __forceinline__ int sobel_mag(int n)
{
    const float f = (float)min(n, 65280);
    float r;
    asm("sqrt.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(f));
    return (int)(r + 0.5f);
}

// ---------------------------------------------------------------------------------
// Sobel: dx = [1,2,1]^T (x) [-1,0,1], dy = [-1,0,1]^T (x) [1,2,1] (correlation,
// A9), fused with the magnitude point operator.  Exact integers.
// ---------------------------------------------------------------------------------
struct OpSobel {
    using Tin = uint8_t;
    static constexpr int NIN = 1, PX = kPxSobel, HX = 1, HY = 1, MH = 3, SEGW = PX + 2;
    static constexpr int PFMAX = kPfSub;  // rows loaded ahead (latency hiding)
    static constexpr bool ROW_DIRECT = false;
    static constexpr bool SHFL_HALO = false;  // shuffle halo measured slower
    struct Params {
        Geom g;
        const uint8_t *in[1];
        uint8_t cval;
        int16_t *dx, *dy;
        uint8_t *mag;
    };
    struct H { int sm[PX], df[PX]; };
    using A = AccI<PX, 2>;
    __host__ __device__ static constexpr bool col_used(int) { return true; }
    __host__ __device__ static constexpr bool row_used(int) { return true; }
    __device__ __forceinline__ static void zero(A &a)
    {
#pragma unroll
        for (int e = 0; e < PX; ++e) a.v[0][e] = a.v[1][e] = 0;
    }
    __device__ __forceinline__ static void hrow(const Params &, const uint8_t (&seg)[1][SEGW], H &h)
    {
#pragma unroll
        for (int e = 0; e < PX; ++e) {
            const int a = seg[0][e], b = seg[0][e + 1], c = seg[0][e + 2];
            h.sm[e] = a + 2 * b + c;
            h.df[e] = c - a;
        }
    }
    template <bool FIRST>
    __device__ __forceinline__ static void vacc(const Params &, int j, const H &h, A &a)
    {
#pragma unroll
        for (int e = 0; e < PX; ++e) {
            a.v[0][e] = (FIRST ? 0 : a.v[0][e]) + (j == 1 ? 2 : 1) * h.df[e];
            if (FIRST) a.v[1][e] = (j - 1) * h.sm[e];
            else if (j != 1) a.v[1][e] += (j - 1) * h.sm[e];
        }
    }
    template <int CK>
    __device__ __forceinline__ static void store(const Params &p, const A &a, int x0, int y)
    {
        const size_t off = (ptrdiff_t)(y - p.g.oy0) * p.g.out_pitch;
        if (p.dx) {
            int16_t o[PX];
#pragma unroll
            for (int e = 0; e < PX; ++e) o[e] = (int16_t)a.v[0][e];
            store_px<CK, int16_t, PX>(p.dx + off, x0, p.g.w, p.g.vec_out, o);
        }
        if (p.dy) {
            int16_t o[PX];
#pragma unroll
            for (int e = 0; e < PX; ++e) o[e] = (int16_t)a.v[1][e];
            store_px<CK, int16_t, PX>(p.dy + off, x0, p.g.w, p.g.vec_out, o);
        }
        if (p.mag) {
            uint8_t o[PX];
#pragma unroll
            for (int e = 0; e < PX; ++e)
                o[e] = (uint8_t)sobel_mag(a.v[0][e] * a.v[0][e] + a.v[1][e] * a.v[1][e]);
            store_px<CK, uint8_t, PX>(p.mag + off, x0, p.g.w, p.g.vec_out, o);
        }
    }
};

// Laplace 5x5 (a8): box sum minus 25 x centre (== ones mask with centre -24).
// One accumulator per output (the centre term enters with the centre row, j == 2), and
// the horizontal 5-sums slide (2 ops per pixel after the first).
struct OpLaplace5 {
    using Tin = uint8_t;
    static constexpr int NIN = 1, PX = kPxLaplace, HX = 2, HY = 2, MH = 5, SEGW = PX + 4;
    static constexpr int PFMAX = kPfSub;  // rows loaded ahead (latency hiding)
    static constexpr bool ROW_DIRECT = false;
    static constexpr bool SHFL_HALO = false;  // shuffle halo measured slower
    struct Params {
        Geom g;
        const uint8_t *in[1];
        uint8_t cval;
        uint8_t *out;
    };
    struct H { int box[PX], ctr[PX]; };
    using A = AccI<PX, 1>;
    __host__ __device__ static constexpr bool col_used(int) { return true; }
    __host__ __device__ static constexpr bool row_used(int) { return true; }
    __device__ __forceinline__ static void zero(A &a)
    {
#pragma unroll
        for (int e = 0; e < PX; ++e) a.v[0][e] = 0;
    }
    __device__ __forceinline__ static void hrow(const Params &, const uint8_t (&seg)[1][SEGW], H &h)
    {
        int s = 0;
#pragma unroll
        for (int i = 0; i < 5; ++i) s += seg[0][i];
        h.box[0] = s;
#pragma unroll
        for (int e = 1; e < PX; ++e) {
            s += (int)seg[0][e + 4] - (int)seg[0][e - 1];
            h.box[e] = s;
        }
#pragma unroll
        for (int e = 0; e < PX; ++e) h.ctr[e] = seg[0][e + 2];
    }
    template <bool FIRST>
    __device__ __forceinline__ static void vacc(const Params &, int j, const H &h, A &a)
    {
#pragma unroll
        for (int e = 0; e < PX; ++e)
            a.v[0][e] = (FIRST ? 0 : a.v[0][e]) + (j == 2 ? h.box[e] - 25 * h.ctr[e] : h.box[e]);
    }
    template <int CK>
    __device__ __forceinline__ static void store(const Params &p, const A &a, int x0, int y)
    {
        uint8_t o[PX];
#pragma unroll
        for (int e = 0; e < PX; ++e) o[e] = sat_u8(a.v[0][e]);
        store_px<CK, uint8_t, PX>(p.out + (ptrdiff_t)(y - p.g.oy0) * p.g.out_pitch, x0, p.g.w, p.g.vec_out, o);
    }
};

// Harris over (dx, dy) int16 (a10; BASELINE configs[2]): 3x3, w = [1,2,1](x)[1,2,1].
// Exact in floating point: |dx|, |dy| <= 1020, so every product (<= 1020^2) and every
// weighted sum Sxx, Syy, |Sxy| <= 16 * 1020^2 = 16,646,400 < 2^24 is an integer that f32
// represents exactly, in any summation order.  The response
// R25 = 25 (Sxx Syy - Sxy^2) - (Sxx + Syy)^2 has every intermediate below 2^53 in
// magnitude (25 * Sxx * Syy <= 6.9e15), so f64 evaluates it exactly; the comparison with
// the int64 threshold is exact after clamping it to +-2^53.  Same bits as the int64
// definition (oracle) by construction.
__device__ __forceinline__ float i16_to_f32(int x)
{
    // 1.5 * 2^23 + x has the integer x in its low mantissa bits for |x| < 2^22
    return __int_as_float(0x4B400000 + x) - 12582912.0f;
}

struct OpHarris {
    using Tin = int16_t;
    static constexpr int NIN = 2, PX = kPxI16, HX = 1, HY = 1, MH = 3, SEGW = PX + 2;
    static constexpr int PFMAX = kPfSub;  // rows loaded ahead (latency hiding)
    static constexpr bool ROW_DIRECT = false;
    static constexpr bool SHFL_HALO = false;  // shuffle halo measured slower
    struct Params {
        Geom g;
        const int16_t *in[2];
        int16_t cval;
        long long thr;
        uint8_t *out;
    };
    struct H { float xx[PX], yy[PX], xy[PX]; };
    struct A { float v[3][PX]; };
    __host__ __device__ static constexpr bool col_used(int) { return true; }
    __host__ __device__ static constexpr bool row_used(int) { return true; }
    __device__ __forceinline__ static void zero(A &a)
    {
#pragma unroll
        for (int e = 0; e < PX; ++e) a.v[0][e] = a.v[1][e] = a.v[2][e] = 0.f;
    }
    __device__ __forceinline__ static void hrow(const Params &, const int16_t (&seg)[2][SEGW], H &h)
    {
        float pxx[SEGW], pyy[SEGW], pxy[SEGW];
#pragma unroll
        for (int k = 0; k < SEGW; k += 2) {
            const float gx0 = i16_to_f32(seg[0][k]), gx1 = i16_to_f32(seg[0][k + 1]);
            const float gy0 = i16_to_f32(seg[1][k]), gy1 = i16_to_f32(seg[1][k + 1]);
            pxx[k] = gx0 * gx0;
            pxx[k + 1] = gx1 * gx1;
            pyy[k] = gy0 * gy0;
            pyy[k + 1] = gy1 * gy1;
            pxy[k] = gx0 * gy0;
            pxy[k + 1] = gx1 * gy1;
        }
#pragma unroll
        for (int e = 0; e < PX; ++e) {
            h.xx[e] = fmaf(2.f, pxx[e + 1], pxx[e]) + pxx[e + 2];
            h.yy[e] = fmaf(2.f, pyy[e + 1], pyy[e]) + pyy[e + 2];
            h.xy[e] = fmaf(2.f, pxy[e + 1], pxy[e]) + pxy[e + 2];
        }
    }
    template <bool FIRST>
    __device__ __forceinline__ static void vacc(const Params &, int j, const H &h, A &a)
    {
        const float wj = (j == 1) ? 2.f : 1.f;
#pragma unroll
        for (int e = 0; e < PX; e += 2) {
            if (FIRST) {
                a.v[0][e] = h.xx[e]; a.v[0][e + 1] = h.xx[e + 1];
                a.v[1][e] = h.yy[e]; a.v[1][e + 1] = h.yy[e + 1];
                a.v[2][e] = h.xy[e]; a.v[2][e + 1] = h.xy[e + 1];
            } else {
                fma2(a.v[0][e], a.v[0][e + 1], wj, h.xx[e], h.xx[e + 1]);
                fma2(a.v[1][e], a.v[1][e + 1], wj, h.yy[e], h.yy[e + 1]);
                fma2(a.v[2][e], a.v[2][e + 1], wj, h.xy[e], h.xy[e + 1]);
            }
        }
    }
    template <int CK>
    __device__ __forceinline__ static void store(const Params &p, const A &a, int x0, int y)
    {
        const double thr = (double)max(-9007199254740992ll, min(9007199254740992ll, p.thr));  // +-2^53
        uint8_t o[PX];
#pragma unroll
        for (int e = 0; e < PX; ++e) {
            const double sxx = a.v[0][e], syy = a.v[1][e], sxy = a.v[2][e];
            const double det = fma(-sxy, sxy, sxx * syy);      // exact: all terms < 2^49
            const double tr = sxx + syy;                        // exact
            const double r25 = fma(25.0, det, -(tr * tr));      // exact: |.| < 2^53
            o[e] = r25 > thr ? 255 : 0;
        }
        store_px<CK, uint8_t, PX>(p.out + (ptrdiff_t)(y - p.g.oy0) * p.g.out_pitch, x0, p.g.w, p.g.vec_out, o);
    }
};

// Atrous pass, dilation D (P:L355 Night filter; a12, A26): h = [1,2,1]/4 at taps
// -D, 0, +D in x and y.  Only the used columns/rows are loaded (sparse window, the
// "holes"); ISP bounds use the effective half-width D.  Optional fused tone map.
template <int D>
struct OpAtrous {
    using Tin = float;
    static constexpr int NIN = 1, PX = 4, HX = D, HY = D, MH = 2 * D + 1, SEGW = PX + 2 * D;
    static constexpr int PFMAX = 0;
    static constexpr bool ROW_DIRECT = true;
    static constexpr bool SHFL_HALO = false;
    static constexpr int NTAPS_Y = 3;
    __host__ __device__ static constexpr int vtap(int t) { return (t - 1) * D; }
    struct Params {
        Geom g;
        const float *in[1];
        float cval;
        float *out;
        int tonemap;
    };
    struct H { float v[PX]; };
    using A = AccF<PX>;
    __host__ __device__ static constexpr bool col_used(int k)
    {
        return k < PX || (k >= D && k < D + PX) || (k >= 2 * D && k < 2 * D + PX);
    }
    __host__ __device__ static constexpr bool row_used(int j) { return j == 0 || j == D || j == 2 * D; }
    __device__ __forceinline__ static void zero(A &a)
    {
#pragma unroll
        for (int e = 0; e < PX; ++e) a.v[e] = 0.f;
    }
    __device__ __forceinline__ static void hrow(const Params &, const float (&seg)[1][SEGW], H &h)
    {
#pragma unroll
        for (int e = 0; e < PX; ++e) h.v[e] = fmaf(0.25f, seg[0][e + 2 * D], fmaf(0.5f, seg[0][e + D], 0.25f * seg[0][e]));
    }
    template <bool FIRST>
    __device__ __forceinline__ static void vacc(const Params &, int j, const H &h, A &a)
    {
        const float wj = (j == D) ? 0.5f : 0.25f;
#pragma unroll
        for (int e = 0; e < PX; ++e) a.v[e] = fmaf(wj, h.v[e], a.v[e]);
    }
    template <int CK>
    __device__ __forceinline__ static void store(const Params &p, const A &a, int x0, int y)
    {
        float o[PX];
#pragma unroll
        for (int e = 0; e < PX; ++e) o[e] = p.tonemap ? a.v[e] / (1.0f + a.v[e]) : a.v[e];
        store_px<CK, float, PX>(p.out + (ptrdiff_t)(y - p.g.oy0) * p.g.out_pitch, x0, p.g.w, p.g.vec_out, o);
    }
};

}  // namespace ispk
