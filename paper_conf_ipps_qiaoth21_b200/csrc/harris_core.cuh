// harris_core.cuh -- the exact Harris decision R25 > thr (a10, reading A27 / A33) shared by
// the tile (tile_u8.cu) and band (band_u8.cu) kernels: packed FP32x2 helpers, the f32
// evaluation with its rigorous error bound and the exact f64 fallback.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

namespace {

__device__ __forceinline__ float2 f2(float a, float b) { return make_float2(a, b); }
// packed FP32x2 (sm_100 FFMA2 / FMUL2 / FADD2) through the CUDA builtins, so the compiler
// allocates the register pairs itself (the inline-asm form forced pair-building moves)
__device__ __forceinline__ float2 mul2(float2 a, float2 b) { return __fmul2_rn(a, b); }
__device__ __forceinline__ float2 fma2(float2 a, float2 b, float2 c) { return __ffma2_rn(a, b, c); }
__device__ __forceinline__ float2 add2(float2 a, float2 b) { return __fadd2_rn(a, b); }

__device__ __noinline__ int harris_exact(float sxx, float syy, float sxy, double thr)
{
    const double dx = sxx, dy = syy, dz = sxy;
    const double dd = fma(-dz, dz, dx * dy), tr = dx + dy;
    return fma(25.0, dd, -(tr * tr)) > thr ? 255 : 0;
}

// R25 > thr for two pixels: f32 fast path with |R_f - R| <= 2^-17 (p + q + t^2), exact f64
// when the bound cannot decide
__device__ __forceinline__ void harris2(float2 sxx, float2 syy, float2 sxy, float thr_f, float thr_err, double thr,
                                        int &o0, int &o1)
{
    const float2 pp = mul2(sxx, syy), q = mul2(sxy, sxy);
    const float2 det = fma2(f2(-sxy.x, -sxy.y), sxy, pp);
    const float2 t = add2(sxx, syy);
    const float2 tt = mul2(t, t);
    const float2 R = fma2(f2(25.f, 25.f), det, f2(-tt.x, -tt.y));
    const float2 bnd = add2(add2(pp, q), tt);
    // (1 + 2^-10) x the bound: |d| >= b decides strictly; b = 0 only for all-zero sums and
    // thr = 0, where R_f = R25 = 0 is exact (flat areas never take the slow path)
    const float b0 = fmaf(bnd.x, 7.6368451118469238281e-06f, thr_err), b1 = fmaf(bnd.y, 7.6368451118469238281e-06f, thr_err);
    const float d0 = R.x - thr_f, d1 = R.y - thr_f;
    o0 = d0 > 0.f ? 255 : 0;
    o1 = d1 > 0.f ? 255 : 0;
    const bool u0 = fabsf(d0) < b0, u1 = fabsf(d1) < b1;
    if (__any_sync(0xffffffffu, u0 || u1)) {
        if (u0) o0 = bnd.x == 0.f ? (0.0 > thr ? 255 : 0) : harris_exact(sxx.x, syy.x, sxy.x, thr);
        if (u1) o1 = bnd.y == 0.f ? (0.0 > thr ? 255 : 0) : harris_exact(sxx.y, syy.y, sxy.y, thr);
    }
}

// |(float)thr - thr| <= 2^-24 |thr| < 2^-23 |thr_f|, inflated by (1 + 2^-10) like the bound
__host__ __device__ __forceinline__ float thr_bound(float thr_f) { return 1.1932570487260818e-07f * fabsf(thr_f); }

// int16 -> exact float (|v| < 2^22): 1.5 * 2^23 + v has v in its low mantissa bits
__device__ __forceinline__ float i2f(int v) { return __int_as_float(0x4B400000 + v) - 12582912.0f; }


}  // namespace
