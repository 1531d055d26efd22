// band_u8.cu -- warp-strip streaming ISP kernels for the cfg3 u8 operators (round 3): the
// ISP_TMA variant of isp_laplace5_u8 (a8) and isp_harris_u8 (a10).
//
// Partition (Listing 3, at warp granularity as in Listing 5): the
// image is cut into vertical strips of 32 lanes x 4*NW pixels (one warp each; NW = 2 or 4 words) and horizontal
// bands of rows (balanced over one wave of CTAs).  A warp's region follows from whether
// its strip reaches past the left / right edge and its band past the top / bottom edge
// within the window's reach -- warp-uniform -- so every warp runs a body specialised to
// exactly those checks ("fat kernel"); Body warps run none.
//
// Each warp streams the input rows of its band through its own shared-memory ring with
// cp.async (4*NW bytes per lane; the strip's two 4-byte halo words by lanes 0 and 31,
// predicated), D rows
// in flight, and keeps the per-row horizontal 5-sums in a register ring:
//   * horizontal 5-sums directly as 16-bit pair lanes: with E_k = (b_k, b_k+2) and
//     O_k = (b_k+1, b_k+3) (byte permutes of the lane's words and funnel shifts across them),
//     (H0, H2) = S + E_-2 and (H1, H3) = S + O_2 with S = O_-2 + E_0 + O_0 + E_2;
//   * the 5-row box as a running sum on 16-bit pair lanes (pixels (0,2) / (1,3) of each
//     4-pixel group), biased by 6400 = 0x1900 so that clamp(box - 25 c, 0, 255) is a
//     u16x2 max / min against 0x1900 / 0x19FF and the result is the low byte of each lane.
// Border handling lives only in the region bodies: T / B warps map their out-of-image
// rows through the pattern once per row (Constant: the row is C), L / R warps fix the two
// halo bytes beyond the edge in registers (Repeat: the edge lane copies the wrapped word).
// Results are the oracle's bit for bit (exact integer arithmetic).
#include <cuda_runtime.h>
#include <stdint.h>

#include <algorithm>
#include <cmath>
#include <cstdlib>

#include "../../include/isp.h"
#include "internal.h"
#include "harris_core.cuh"
#include "band_common.cuh"

namespace {

#ifndef BAND_LAP_D
#define BAND_LAP_D 5
#endif
constexpr int LD = BAND_LAP_D;             // rows in flight per warp
static_assert(LR >= LD + 1, "ring too small");


// NW words (4 pixels each) per lane
template <int NW> struct BandShape {
    static constexpr int LPX = 4 * NW;           // pixels per lane
    static constexpr int STRIP = 32 * LPX;       // columns per warp
    static constexpr int SLOT = 32 + STRIP;      // [12,16) left halo word, [16,16+STRIP) strip, then right
    static constexpr int MINB = NW == 2 ? 8 : 5; // resident CTAs per SM (register cap)
};

struct LapBandParams {
    BandGeom g;
    const uint8_t *img;
    uint8_t *out;
    uint32_t cword;  // the constant in all four bytes
};

// cp.async of the lane's NW words, predicated on the lane (lanes past the image copy
// nothing, so the halo words stored in their positions survive)
template <int NW>
__device__ __forceinline__ void cpa_own(uint32_t dst, const void *src, uint32_t on)
{
    if constexpr (NW == 4)
        asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %2, 0;\n\t@q cp.async.cg.shared.global [%0], [%1], 16;\n\t}" ::"r"(dst),
                     "l"(src), "r"(on)
                     : "memory");
    else
        asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %2, 0;\n\t@q cp.async.ca.shared.global [%0], [%1], 8;\n\t}" ::"r"(dst),
                     "l"(src), "r"(on)
                     : "memory");
}
template <int NW>
__device__ __forceinline__ void lds_own(uint32_t a, uint32_t (&w)[NW])
{
    if constexpr (NW == 4)
        asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(w[0]), "=r"(w[1]), "=r"(w[2]), "=r"(w[3]) : "r"(a)
                     : "memory");
    else
        asm volatile("ld.shared.v2.u32 {%0, %1}, [%2];" : "=r"(w[0]), "=r"(w[1]) : "r"(a) : "memory");
}
// 16-bit pair lanes of a word: (b0, b2) and (b1, b3)
__device__ __forceinline__ uint32_t ev(uint32_t w) { return __byte_perm(w, 0u, 0x4240); }
__device__ __forceinline__ uint32_t od(uint32_t w) { return __byte_perm(w, 0u, 0x4341); }

// One warp's band: input rows y0-2 .. y0+rows+1 streamed through the warp's ring (shared
// address `ring`, LR slots), LD rows in flight.  Region handling (Listing 3 per warp):
//   * T / B (CY): rows outside the image are mapped through the pattern when they are
//     copied, once per row (Constant: the staged row is C);
//   * L / R (cl / cr): only the edge lanes' halo words differ -- the wrapped word is copied
//     (Repeat), the constant pre-stored (Constant), or the word is rebuilt from the lane's
//     own edge bytes by a byte permute chosen once per warp (Clamp / Mirror; every other
//     lane's selector is the identity), so the row loop itself carries no checks at all.
template <int NW, bool CY>
__device__ __forceinline__ void lap_band_body(const LapBandParams &p, uint32_t ring, int xs0, int y0, int rows,
                                              int lane, bool cl, bool cr)
{
    using B = BandShape<NW>;
    constexpr int LPX = B::LPX, STRIP = B::STRIP, SLOT = B::SLOT;
    const BandGeom &g = p.g;
    const int x = xs0 + LPX * lane;
    const bool active = !cr || x < g.w;
    const bool redge = cr && x + LPX == g.w;   // the image's last lane (R region)
    const int nin = rows + 4;                  // >= 10 (bands of >= 6 rows)
    const uint32_t loff = LPX * lane;
    // copies per row: the lane's NW words (none past the image) and two predicated
    // 4-byte halo copies -- A: lane 0, the strip's left word (L, Repeat: the wrapped word
    // w-4..w-1); B: lane 31 the strip's right word, or (R, Repeat) the last lane the
    // wrapped word 0..3 into its right neighbour's position
    int acol = xs0 - 4, bcol = xs0 + STRIP;
    uint32_t aon = lane == 0 && (!cl || g.mode == ISP_REPEAT), bdst = 16 + STRIP, bon = !cr && lane == 31;
    if (cl) acol = g.w - 4;
    if (redge && g.mode == ISP_REPEAT) { bon = 1; bcol = 0; bdst = 16 + LPX * (lane + 1); }
    // halo selectors: W[0] = prmt(W[0], W[1], sl_), W[NW+1] = prmt(W[NW+1], W[NW], sr_)
    uint32_t sl_ = 0x3210, sr_ = 0x3210;
    if (cl && lane == 0) sl_ = g.mode == ISP_CLAMP ? 0x4444 : g.mode == ISP_MIRROR ? 0x4500 : 0x3210;
    if (redge) sr_ = g.mode == ISP_CLAMP ? 0x7777 : g.mode == ISP_MIRROR ? 0x0067 : 0x3210;
    if (g.mode == ISP_CONSTANT) {   // the halo positions no copy writes hold C in every slot
        for (int j = 0; j < LR; ++j) {
            if (cl && lane == 0) sts32(ring + j * SLOT + 12, p.cword);
            if (redge) sts32(ring + j * SLOT + 16 + LPX * (lane + 1), p.cword);
        }
    }
    const int mcol = active ? x : 0;
    const uint8_t *nrp = p.img + (ptrdiff_t)(y0 - 2) * g.pitch;   // next row to issue (unmapped)
    auto issue = [&](int j, uint32_t slot) {
        const uint8_t *rp = nrp;
        if constexpr (CY) {   // T / B regions: the row through the pattern, once per row
            const int yy = map_row1<true>(y0 - 2 + j, g.h, g.mode);
            if (yy < 0) {     // Constant: the whole staged row is C
#pragma unroll
                for (int q = 0; q < NW; ++q) sts32(slot + 16 + loff + 4 * q, p.cword);
                if (lane == 0) sts32(slot + 12, p.cword);
                if (lane == 31) sts32(slot + 16 + STRIP, p.cword);
                return;
            }
            rp = p.img + (size_t)yy * g.pitch;
        }
        cpa_own<NW>(slot + 16 + loff, rp + mcol, active);
        cpa4p(slot + 12, rp + acol, aon);
        cpa4p(slot + bdst, rp + bcol, bon);
    };
#pragma unroll
    for (int j = 0; j < LD; ++j) {
        issue(j, ring + j * SLOT);
        nrp += g.pitch;
        cpa_commit();
    }
    // H ring: horizontal 5-sums of the last five rows as pair lanes, per 4-pixel group g
    // (E_g, O_g) = ((H_4g, H_4g+2), (H_4g+1, H_4g+3)); box = sum of the ring + bias 6400
    uint32_t hr[5][2 * NW] = {};
    uint32_t box[2 * NW];
#pragma unroll
    for (int q = 0; q < 2 * NW; ++q) box[q] = 0x19001900u;
    uint32_t c1[NW] = {}, c2[NW] = {};   // own words of rows i-1, i-2 (the centre row)
    uint8_t *orow = p.out + (size_t)y0 * g.out_pitch + x;
#pragma unroll 1
    for (int i0 = 0; i0 < nin; i0 += 5) {
#pragma unroll
        for (int k = 0; k < 5; ++k) {
            const int i = i0 + k;
            if (i < nin) {
                cpa_wait<LD - 1>();
                __syncwarp();
                const uint32_t sl = ring + (i & (LR - 1)) * SLOT + loff;
                uint32_t W[NW + 2];   // W[0] = left halo word, W[1..NW] own, W[NW+1] right
                lds_own<NW>(sl + 16, *reinterpret_cast<uint32_t(*)[NW]>(&W[1]));
                W[0] = __byte_perm(lds32(sl + 12), W[1], sl_);
                W[NW + 1] = __byte_perm(lds32(sl + 16 + LPX), W[NW], sr_);
                // horizontal 5-sums on pair lanes: E_k = (b_k, b_k+2), O_k = (b_k+1, b_k+3);
                // group g (pixels 4g..4g+3): (H,H+2) = S + E_-2, (H+1,H+3) = S + O_2 with
                // S = O_-2 + E_0 + O_0 + E_2 (offsets relative to 4g); F_g = bytes 4g-2..4g+1
                uint32_t Ef[NW + 1], Of[NW + 1];
#pragma unroll
                for (int q = 0; q <= NW; ++q) {
                    const uint32_t F = __funnelshift_r(W[q], W[q + 1], 16);
                    Ef[q] = ev(F);
                    Of[q] = od(F);
                }
                uint32_t hn[2 * NW];
#pragma unroll
                for (int q = 0; q < NW; ++q) {
                    const uint32_t S = Of[q] + ev(W[q + 1]) + od(W[q + 1]) + Ef[q + 1];
                    hn[2 * q] = S + Ef[q];
                    hn[2 * q + 1] = S + Of[q + 1];
                }
                // box of rows i-4..i: + H(i) - H(i-5) (the ring slot being replaced; zero
                // for i < 5)
#pragma unroll
                for (int q = 0; q < 2 * NW; ++q) {
                    box[q] = box[q] + hn[q] - hr[k][q];
                    hr[k][q] = hn[q];
                }
                if (i >= 4) {
                    // output row y0 + i - 4: clamp(box - 25 c, 0, 255), c = row i - 2
                    uint32_t o[NW];
#pragma unroll
                    for (int q = 0; q < NW; ++q) {
                        uint32_t vE = box[2 * q] - 25u * ev(c2[q]), vO = box[2 * q + 1] - 25u * od(c2[q]);
                        asm("max.u16x2 %0, %0, %1;" : "+r"(vE) : "r"(0x19001900u));
                        asm("min.u16x2 %0, %0, %1;" : "+r"(vE) : "r"(0x19FF19FFu));
                        asm("max.u16x2 %0, %0, %1;" : "+r"(vO) : "r"(0x19001900u));
                        asm("min.u16x2 %0, %0, %1;" : "+r"(vO) : "r"(0x19FF19FFu));
                        o[q] = __byte_perm(vE, vO, 0x6240);
                    }
                    if (active) {
                        if constexpr (NW == 4) *reinterpret_cast<uint4 *>(orow) = make_uint4(o[0], o[1], o[2], o[3]);
                        else *reinterpret_cast<uint2 *>(orow) = make_uint2(o[0], o[1]);
                    }
                    orow += g.out_pitch;
                }
#pragma unroll
                for (int q = 0; q < NW; ++q) {
                    c2[q] = c1[q];
                    c1[q] = W[q + 1];
                }
                // refill: row i + LD into the slot of row i + LD - LR (last read at i - 1)
                if (i + LD < nin) issue(i + LD, ring + ((i + LD) & (LR - 1)) * SLOT);
                nrp += g.pitch;
                cpa_commit();
            }
        }
    }
}

template <int NW>
__global__ void __launch_bounds__(NTB, BandShape<NW>::MINB) k_lap_band(const __grid_constant__ LapBandParams p)
{
    using B = BandShape<NW>;
    __shared__ __align__(16) uint8_t rings[BW][LR * B::SLOT];
    asm volatile("griddepcontrol.wait;" ::: "memory");
    asm volatile("griddepcontrol.launch_dependents;");
    const BandGeom &g = p.g;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int gx = (int)blockIdx.x % g.ngx, band = (int)blockIdx.x / g.ngx;
    const int s = gx * BW + warp;
    if (s >= g.nstrip) return;
    int y0, y1;
    band_rows(band, g.nband, g.h, y0, y1);
    const int xs0 = s * B::STRIP;
    // region of this warp (Listing 3 on strip / band indices, warp-uniform): T / B warps run
    // the row-mapping body, L / R warps set their edge lanes' halo handling
    const bool cl = s < g.sx0, cr = s >= g.sx1, cy = band < g.by0 || band >= g.by1;
    const uint32_t ring = su32(rings[warp]);
    if (cy) lap_band_body<NW, true>(p, ring, xs0, y0, y1 - y0, lane, cl, cr);
    else lap_band_body<NW, false>(p, ring, xs0, y0, y1 - y0, lane, cl, cr);
}


// ------------------------------------------------------------------------------ Harris
// Same skeleton over the int16 derivative images (a10): 4 pixels per lane (one 8-byte word
// pair per image), strips of 128 columns, the ring slot holding the dx row then the dy row
// (each with its two halo words), rows y0-1 .. y0+rows.  Per row the lane forms the
// horizontal [1,2,1] sums of dx^2, dy^2, dx*dy as exact FP32x2 pairs (E = pixels (0,2),
// O = (1,3)), keeps the last three in a register ring and decides R25 > thr exactly
// (harris_core.cuh).  Border handling as in the Laplace body: rows mapped at copy time,
// the edge lanes' halo words by per-warp selectors (Constant: C pre-stored).
struct HarBandParams {
    BandGeom g;
    const int16_t *dx, *dy;
    uint8_t *out;
    uint32_t cword;   // the constant in both int16 halves
    double thr;
    float thr_f, thr_err;
};

// G groups of 4 pixels per lane: strips of 128 G columns; a slot holds the dx row then the
// dy row, each [12,16) left halo word, [16, 16 + 256 G) strip, then the right halo word
template <int G> struct HarShape {
    static constexpr int STRIP = 128 * G;
    static constexpr int IMG = 32 + 2 * STRIP;
    static constexpr int SLOT = 2 * IMG;
};
constexpr int HLD = 5;                      // rows in flight per warp

struct HRow { float2 xxE, xxO, yyE, yyO, xyE, xyO; };

// int16 halves (sa of a, sb of b: 0x7610 = low half, 0x7632 = high half) as an exact float
// pair: the biased halves land in the mantissa of 2^23, one packed subtract removes 2^23 + 32768
__device__ __forceinline__ float2 i16pair(uint32_t a, uint32_t sa, uint32_t b, uint32_t sb)
{
    const float2 r = make_float2(__uint_as_float(__byte_perm(a ^ 0x80008000u, 0x4B000000u, sa)),
                                 __uint_as_float(__byte_perm(b ^ 0x80008000u, 0x4B000000u, sb)));
    return add2(r, f2(-8421376.0f, -8421376.0f));
}

// Horizontal [1,2,1] sums of xx, yy, xy for pixels 0..3 from the words (L, X0, X1, R) of dx
// and dy (L = pixels -2,-1; R = 4,5) through the pairs A = (p-1, p1), E, O, B = (p2, p4)
// (har_hrow_f: no pair shuffling).  Products of integers <= 1020 are exact in f32.
__device__ __forceinline__ HRow har_hrow_f(float2 xA, float2 xE, float2 xO, float2 xB, float2 yA, float2 yE, float2 yO,
                                           float2 yB);
__device__ __forceinline__ HRow har_hrow(uint32_t XL, uint32_t X0, uint32_t X1, uint32_t XR, uint32_t YL, uint32_t Y0,
                                         uint32_t Y1, uint32_t YR)
{
    const float2 xA = i16pair(XL, 0x7632, X0, 0x7632), xE = i16pair(X0, 0x7610, X1, 0x7610);
    const float2 xO = i16pair(X0, 0x7632, X1, 0x7632), xB = i16pair(X1, 0x7610, XR, 0x7610);
    const float2 yA = i16pair(YL, 0x7632, Y0, 0x7632), yE = i16pair(Y0, 0x7610, Y1, 0x7610);
    const float2 yO = i16pair(Y0, 0x7632, Y1, 0x7632), yB = i16pair(Y1, 0x7610, YR, 0x7610);
    return har_hrow_f(xA, xE, xO, xB, yA, yE, yO, yB);
}

// R25 > thr for a pixel pair, exact (reading A33).  f32 evaluation
// R = 25 (Sxx Syy - Sxy^2) - t^2 with t = Sxx + Syy; its error is at most
// 2^-24 (76 Sxx Syy + 51 Sxy^2 + 4.1 t^2)(1 + O(2^-24)) <= 2^-24 * 36 t^2, since
// Sxx Syy <= t^2 / 4 (AM-GM) and Sxy^2 <= Sxx Syy (Cauchy-Schwarz, positive weights); the
// decision bound b = 1.5 * 2^-17 * fl(t^2) + |fl(thr) - thr| (= 2^-24 * 192 t^2) covers it
// five times over.  Pixels within the bound take the exact f64 form (t = 0: R25 = 0).
__device__ __forceinline__ void harris2p(float2 sxx, float2 syy, float2 sxy, float thr_f, float thr_err, double thr,
                                         uint32_t &o0, uint32_t &o1)
{
    const float2 pp = mul2(sxx, syy);
    const float2 det = fma2(f2(-sxy.x, -sxy.y), sxy, pp);
    const float2 t = add2(sxx, syy);
    const float2 tt = mul2(t, t);
    const float2 R = fma2(f2(25.f, 25.f), det, f2(-tt.x, -tt.y));
    // b = (1 + 2^-10) x the bound, so that |d| >= b decides strictly (and b = 0 only for
    // t = 0 and thr = 0, where R_f = R25 = 0 is exact: flat areas never take the slow path)
    const float2 b = fma2(tt, f2(1.14552676677703857421875e-05f, 1.14552676677703857421875e-05f), f2(thr_err, thr_err));
    const float2 d = add2(R, f2(-thr_f, -thr_f));
    o0 = d.x > 0.f ? 255u : 0u;
    o1 = d.y > 0.f ? 255u : 0u;
    const bool u0 = fabsf(d.x) < b.x, u1 = fabsf(d.y) < b.y;   // undecided by the bound
    if (__any_sync(0xffffffffu, u0 || u1)) {
        if (u0) o0 = tt.x == 0.f ? (0.0 > thr ? 255u : 0u) : (uint32_t)harris_exact(sxx.x, syy.x, sxy.x, thr);
        if (u1) o1 = tt.y == 0.f ? (0.0 > thr ? 255u : 0u) : (uint32_t)harris_exact(sxx.y, syy.y, sxy.y, thr);
    }
}

// harris2p for the pairs E and O of four pixels with one warp vote (same decisions)
__device__ __forceinline__ uint32_t harris4v(float2 sxxE, float2 syyE, float2 sxyE, float2 sxxO, float2 syyO,
                                             float2 sxyO, float thr_f, float thr_err, double thr)
{
    const float2 c = f2(1.14552676677703857421875e-05f, 1.14552676677703857421875e-05f), te = f2(thr_err, thr_err);
    const float2 ntf = f2(-thr_f, -thr_f), k25 = f2(25.f, 25.f);
    const float2 tE = add2(sxxE, syyE), tO = add2(sxxO, syyO);
    const float2 ttE = mul2(tE, tE), ttO = mul2(tO, tO);
    const float2 RE = fma2(k25, fma2(f2(-sxyE.x, -sxyE.y), sxyE, mul2(sxxE, syyE)), f2(-ttE.x, -ttE.y));
    const float2 RO = fma2(k25, fma2(f2(-sxyO.x, -sxyO.y), sxyO, mul2(sxxO, syyO)), f2(-ttO.x, -ttO.y));
    const float2 bE = fma2(ttE, c, te), bO = fma2(ttO, c, te);
    const float2 dE = add2(RE, ntf), dO = add2(RO, ntf);
    uint32_t h0 = dE.x > 0.f ? 255u : 0u, h2 = dE.y > 0.f ? 255u : 0u;
    uint32_t h1 = dO.x > 0.f ? 255u : 0u, h3 = dO.y > 0.f ? 255u : 0u;
    const bool u0 = fabsf(dE.x) < bE.x, u2 = fabsf(dE.y) < bE.y, u1 = fabsf(dO.x) < bO.x, u3 = fabsf(dO.y) < bO.y;
    if (__any_sync(0xffffffffu, u0 || u1 || u2 || u3)) {
        if (u0) h0 = ttE.x == 0.f ? (0.0 > thr ? 255u : 0u) : (uint32_t)harris_exact(sxxE.x, syyE.x, sxyE.x, thr);
        if (u2) h2 = ttE.y == 0.f ? (0.0 > thr ? 255u : 0u) : (uint32_t)harris_exact(sxxE.y, syyE.y, sxyE.y, thr);
        if (u1) h1 = ttO.x == 0.f ? (0.0 > thr ? 255u : 0u) : (uint32_t)harris_exact(sxxO.x, syyO.x, sxyO.x, thr);
        if (u3) h3 = ttO.y == 0.f ? (0.0 > thr ? 255u : 0u) : (uint32_t)harris_exact(sxxO.y, syyO.y, sxyO.y, thr);
    }
    return __byte_perm(__byte_perm(h0, h1, 0x0040), __byte_perm(h2, h3, 0x0040), 0x5410);
}

template <int G, bool CY>
__device__ __forceinline__ void har_band_body(const HarBandParams &p, uint32_t ring, int xs0, int y0, int rows,
                                              int lane, bool cl, bool cr)
{
    constexpr int STRIP = HarShape<G>::STRIP, HIMG = HarShape<G>::IMG, HSLOT = HarShape<G>::SLOT, NWD = 2 * G;
    const BandGeom &g = p.g;
    const int x = xs0 + 4 * G * lane;
    const bool active = !cr || x < g.w;
    const bool redge = cr && x + 4 * G == g.w;
    const int nin = rows + 2;   // >= 8
    const uint32_t loff = 8 * G * lane;
    // halo copies (columns, in int16 elements): A = lane 0's left word (L, Repeat: w-2, w-1),
    // B = lane 31's right word, or (R, Repeat) the last lane's wrapped word (0, 1)
    int acol = xs0 - 2, bcol = xs0 + STRIP;
    uint32_t aon = lane == 0 && (!cl || g.mode == ISP_REPEAT), bdst = 16 + 2 * STRIP, bon = !cr && lane == 31;
    if (cl) acol = g.w - 2;
    if (redge && g.mode == ISP_REPEAT) { bon = 1; bcol = 0; bdst = 16 + 8 * G * (lane + 1); }
    // selectors: left word = prmt(loaded, first own word, sl_), right = prmt(loaded, last own word, sr_)
    uint32_t sl_ = 0x3210, sr_ = 0x3210;
    if (cl && lane == 0) sl_ = g.mode == ISP_CLAMP ? 0x5454 : g.mode == ISP_MIRROR ? 0x5476 : 0x3210;
    if (redge) sr_ = g.mode == ISP_CLAMP ? 0x7676 : g.mode == ISP_MIRROR ? 0x5476 : 0x3210;
    if (g.mode == ISP_CONSTANT) {
        for (int j = 0; j < LR; ++j)
            for (int im = 0; im < 2; ++im) {
                if (cl && lane == 0) sts32(ring + j * HSLOT + im * HIMG + 12, p.cword);
                if (redge) sts32(ring + j * HSLOT + im * HIMG + 16 + 8 * G * (lane + 1), p.cword);
            }
    }
    const int mcol = active ? x : 0;
    const size_t pitchb = (size_t)g.pitch * 2;
    const char *nx = reinterpret_cast<const char *>(p.dx) + (ptrdiff_t)(y0 - 1) * (ptrdiff_t)pitchb;
    const char *ny = reinterpret_cast<const char *>(p.dy) + (ptrdiff_t)(y0 - 1) * (ptrdiff_t)pitchb;
    auto issue = [&](int j, uint32_t slot) {
        const char *rx = nx, *ry = ny;
        if constexpr (CY) {
            const int yy = map_row1<true>(y0 - 1 + j, g.h, g.mode);
            if (yy < 0) {   // Constant: both staged rows are C
                for (int im = 0; im < 2; ++im) {
#pragma unroll
                    for (int q = 0; q < NWD; ++q) sts32(slot + im * HIMG + 16 + loff + 4 * q, p.cword);
                    if (lane == 0) sts32(slot + im * HIMG + 12, p.cword);
                    if (lane == 31) sts32(slot + im * HIMG + 16 + 2 * STRIP, p.cword);
                }
                return;
            }
            rx = reinterpret_cast<const char *>(p.dx) + (size_t)yy * pitchb;
            ry = reinterpret_cast<const char *>(p.dy) + (size_t)yy * pitchb;
        }
        cpa_own<NWD>(slot + 16 + loff, rx + 2 * mcol, active);
        cpa_own<NWD>(slot + HIMG + 16 + loff, ry + 2 * mcol, active);
        cpa4p(slot + 12, rx + 2 * acol, aon);
        cpa4p(slot + HIMG + 12, ry + 2 * acol, aon);
        cpa4p(slot + bdst, rx + 2 * bcol, bon);
        cpa4p(slot + HIMG + bdst, ry + 2 * bcol, bon);
    };
#pragma unroll
    for (int j = 0; j < HLD; ++j) {
        issue(j, ring + j * HSLOT);
        nx += pitchb;
        ny += pitchb;
        cpa_commit();
    }
    HRow hr[3][G];
    uint8_t *orow = p.out + (size_t)y0 * g.out_pitch + x;
    const float2 two = f2(2.f, 2.f);
#pragma unroll 1
    for (int i0 = 0; i0 < nin; i0 += 3) {
#pragma unroll
        for (int k = 0; k < 3; ++k) {
            const int i = i0 + k;
            if (i < nin) {
                cpa_wait<HLD - 1>();
                __syncwarp();
                const uint32_t sl = ring + (i & (LR - 1)) * HSLOT + loff;
                uint32_t X[NWD + 2], Y[NWD + 2];   // [0] left halo word, [1..NWD] own, [NWD+1] right
                lds_own<NWD>(sl + 16, *reinterpret_cast<uint32_t(*)[NWD]>(&X[1]));
                lds_own<NWD>(sl + HIMG + 16, *reinterpret_cast<uint32_t(*)[NWD]>(&Y[1]));
                X[0] = __byte_perm(lds32(sl + 12), X[1], sl_);
                Y[0] = __byte_perm(lds32(sl + HIMG + 12), Y[1], sl_);
                X[NWD + 1] = __byte_perm(lds32(sl + 16 + 8 * G), X[NWD], sr_);
                Y[NWD + 1] = __byte_perm(lds32(sl + HIMG + 16 + 8 * G), Y[NWD], sr_);
#pragma unroll
                for (int q = 0; q < G; ++q)
                    hr[k][q] = har_hrow(X[2 * q], X[2 * q + 1], X[2 * q + 2], X[2 * q + 3], Y[2 * q], Y[2 * q + 1],
                                        Y[2 * q + 2], Y[2 * q + 3]);
                if (i >= 2) {
                    // output row y0 + i - 2: rows i-2, i-1, i are hr[k+1], hr[k+2], hr[k] (mod 3)
                    uint32_t o[G];
#pragma unroll
                    for (int q = 0; q < G; ++q) {
                        const HRow &a = hr[(k + 1) % 3][q], &b = hr[(k + 2) % 3][q], &c = hr[k][q];
                        const float2 sxxE = add2(fma2(two, b.xxE, a.xxE), c.xxE), sxxO = add2(fma2(two, b.xxO, a.xxO), c.xxO);
                        const float2 syyE = add2(fma2(two, b.yyE, a.yyE), c.yyE), syyO = add2(fma2(two, b.yyO, a.yyO), c.yyO);
                        const float2 sxyE = add2(fma2(two, b.xyE, a.xyE), c.xyE), sxyO = add2(fma2(two, b.xyO, a.xyO), c.xyO);
                        uint32_t h0, h1, h2, h3;
                        harris2p(sxxE, syyE, sxyE, p.thr_f, p.thr_err, p.thr, h0, h2);
                        harris2p(sxxO, syyO, sxyO, p.thr_f, p.thr_err, p.thr, h1, h3);
                        o[q] = __byte_perm(__byte_perm(h0, h1, 0x0040), __byte_perm(h2, h3, 0x0040), 0x5410);
                    }
                    if (active) {
                        if constexpr (G == 2) *reinterpret_cast<uint2 *>(orow) = make_uint2(o[0], o[1]);
                        else *reinterpret_cast<uint32_t *>(orow) = o[0];
                    }
                    orow += g.out_pitch;
                }
                if (i + HLD < nin) issue(i + HLD, ring + ((i + HLD) & (LR - 1)) * HSLOT);
                nx += pitchb;
                ny += pitchb;
                cpa_commit();
            }
        }
    }
}

template <int G>
__global__ void __launch_bounds__(NTB, G == 1 ? 4 : 3) k_har_band(const __grid_constant__ HarBandParams p)
{
    __shared__ __align__(16) uint8_t rings[BW][LR * HarShape<G>::SLOT];
    asm volatile("griddepcontrol.wait;" ::: "memory");
    asm volatile("griddepcontrol.launch_dependents;");
    const BandGeom &g = p.g;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int gx = (int)blockIdx.x % g.ngx, band = (int)blockIdx.x / g.ngx;
    const int s = gx * BW + warp;
    if (s >= g.nstrip) return;
    int y0, y1;
    band_rows(band, g.nband, g.h, y0, y1);
    const bool cl = s < g.sx0, cr = s >= g.sx1, cy = band < g.by0 || band >= g.by1;
    const uint32_t ring = su32(rings[warp]);
    if (cy) har_band_body<G, true>(p, ring, s * HarShape<G>::STRIP, y0, y1 - y0, lane, cl, cr);
    else har_band_body<G, false>(p, ring, s * HarShape<G>::STRIP, y0, y1 - y0, lane, cl, cr);
}

// pixel groups of 4 per lane of the Harris band launch: 2 unless ISP_HARRIS_G=1
int harris_g()
{
    const char *e = getenv("ISP_HARRIS_G");
    return e && atoi(e) == 1 ? 1 : 2;
}
const void *har_band_fn(int gq) { return gq == 1 ? (const void *)k_har_band<1> : (const void *)k_har_band<2>; }
int har_blocks_per_sm(int gq)
{
    static int nb[3] = {-1, -1, -1};
    if (nb[gq] < 0) {
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb[gq], har_band_fn(gq), NTB, 0) != cudaSuccess) {
            cudaGetLastError();
            nb[gq] = 0;
        }
    }
    return nb[gq];
}


// ------------------------------------------------------------------------------ fused cfg3
// BASELINE configs[2] in one band launch (the ISP_TMA variant of
// isp_pipeline_cfg3_u8): per warp a strip of 128 columns (4 pixels per lane), the u8 rows
// y0-2 .. y0+rows+1 streamed through the cp.async ring once; per row the lane forms the
// byte pair lanes E_k / O_k (as the Laplace body) and from them
//   * Laplace: the horizontal 5-sum pairs, a 5-row running box (ring rotated in registers);
//   * Sobel: horizontal parts s = a + 2b + c and d = c - a for the pairs A = (p-1, p1),
//     E = (p0, p2), O = (p1, p3), B = (p2, p4), biased 16-bit lanes (no borrows); two rows
//     later dx = d + 2d + d and dy = s - s (bias 1024 per lane), as exact floats;
//   * magnitude: sqrt.approx of min(dx^2 + dy^2, 65280) rounded to nearest (DESIGN.md 7c:
//     never within 4.9e-4 of a tie, so it equals round-half-up), read as the low byte;
//   * Harris over the dx / dy IMAGES: horizontal [1,2,1] sums of the products (pairs A..B
//     supply p-1 and p4), a 3-row ring, the exact decision harris2p.
// Border handling: the image pattern for Laplace / Sobel is the staging's (rows mapped at
// copy time, the edge lanes' halo words by selectors); Harris reads dx / dy at REMAPPED
// coordinates, which differ from the shifted window outside the image: the edge lane of an
// L / R warp replaces its dx / dy at column -1 / w by the value at B(-1) / B(w) (Clamp,
// Mirror: its own column 0 / w-1; Constant: the Harris constant; Repeat: the shifted
// window over the periodic image already is dx / dy at the wrapped column), and the band
// holding row 0 / h-1 replaces its ext dx / dy row -1 / h likewise (row 0 / h-1, the
// constant, or Repeat's natural value).  Bit-exact against the oracle composition.
struct FusedBandParams {
    BandGeom g;
    const uint8_t *img;
    uint8_t *mag, *lap, *har;
    int16_t *dx, *dy;
    uint32_t cword;     // the image constant in all four bytes
    float c4;           // 4 hc^2: every [1,2,1] sum of a constant-hc row of products
    float hcf;          // the Harris constant
    double thr;
    float thr_f, thr_err;
};

#ifndef FUSED_FLD
#define FUSED_FLD 5
#endif
#ifndef FUSED_MINB
#define FUSED_MINB 4
#endif
// rows in flight per warp (FLD) and ring slots (FLR >= FLD + 3: rows i-2 .. i+FLD)
constexpr int FSTRIP = 128, FSLOT = 32 + FSTRIP, FLD = FUSED_FLD, FLR = FLD + 3 <= 8 ? 8 : 16;

struct SobH { uint32_t sA, sE, sO, sB, dA, dE, dO, dB; };

// (lanes of x) - bias as floats: 2^23 + lane read from the mantissa, one packed subtract
__device__ __forceinline__ float2 lanes_f(uint32_t x, float bias)
{
    const float2 r = make_float2(__uint_as_float(__byte_perm(x, 0x4B000000u, 0x7610)),
                                 __uint_as_float(__byte_perm(x, 0x4B000000u, 0x7632)));
    return add2(r, f2(-8388608.0f - bias, -8388608.0f - bias));
}

// Horizontal [1,2,1] sums of the products from dx / dy as the pairs A = (p-1, p1), E, O,
// B = (p2, p4): (H0, H2) = A + 2E + O, (H1, H3) = E + 2O + B (no pair shuffling)
__device__ __forceinline__ HRow har_hrow_f(float2 xA, float2 xE, float2 xO, float2 xB, float2 yA, float2 yE, float2 yO,
                                           float2 yB)
{
    const float2 two = f2(2.f, 2.f);
    const float2 xxE = mul2(xE, xE), xxO = mul2(xO, xO), yyE = mul2(yE, yE), yyO = mul2(yO, yO);
    const float2 xyE = mul2(xE, yE), xyO = mul2(xO, yO);
    HRow h;
    h.xxE = add2(fma2(two, xxE, mul2(xA, xA)), xxO);
    h.xxO = add2(fma2(two, xxO, xxE), mul2(xB, xB));
    h.yyE = add2(fma2(two, yyE, mul2(yA, yA)), yyO);
    h.yyO = add2(fma2(two, yyO, yyE), mul2(yB, yB));
    h.xyE = add2(fma2(two, xyE, mul2(xA, yA)), xyO);
    h.xyO = add2(fma2(two, xyO, xyE), mul2(xB, yB));
    return h;
}

// magnitude byte of a pixel from exact float dx, dy
__device__ __forceinline__ uint32_t mag_bits(float n)
{
    float r;
    asm("sqrt.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(fminf(n, 65280.0f)));
    return __float_as_uint(r + 8388608.0f);   // low byte = round(r) <= 255
}

template <bool CY, bool DXY>
__device__ __forceinline__ void fused_band_body(const FusedBandParams &p, uint32_t ring, int xs0, int y0, int rows,
                                                int lane, bool cl, bool cr)
{
    const BandGeom &g = p.g;
    constexpr int LPX = 4;
    const int x = xs0 + LPX * lane;
    const bool active = !cr || x < g.w;
    const bool redge = cr && x + LPX == g.w;
    const int nin = rows + 4;   // >= 10
    const uint32_t loff = LPX * lane;
    // staging as in the Laplace body (one word per lane)
    int acol = xs0 - 4, bcol = xs0 + FSTRIP;
    uint32_t aon = lane == 0 && (!cl || g.mode == ISP_REPEAT), bdst = 16 + FSTRIP, bon = !cr && lane == 31;
    if (cl) acol = g.w - 4;
    if (redge && g.mode == ISP_REPEAT) { bon = 1; bcol = 0; bdst = 16 + LPX * (lane + 1); }
    uint32_t sl_ = 0x3210, sr_ = 0x3210;
    if (cl && lane == 0) sl_ = g.mode == ISP_CLAMP ? 0x4444 : g.mode == ISP_MIRROR ? 0x4500 : 0x3210;
    if (redge) sr_ = g.mode == ISP_CLAMP ? 0x7777 : g.mode == ISP_MIRROR ? 0x0067 : 0x3210;
    if (g.mode == ISP_CONSTANT) {
        for (int j = 0; j < FLR; ++j) {
            if (cl && lane == 0) sts32(ring + j * FSLOT + 12, p.cword);
            if (redge) sts32(ring + j * FSLOT + 16 + LPX * (lane + 1), p.cword);
        }
    }
    // Harris' remapped dx / dy at column -1 (this lane's pixel p-1) / w (pixel p4): 1 = the
    // lane's own column 0 / w-1 (Clamp, Mirror), 2 = the Harris constant (Constant)
    const int rep = g.mode == ISP_REPEAT ? 0 : g.mode == ISP_CONSTANT ? 2 : 1;
    const int ea = cl && lane == 0 ? rep : 0, eb = redge ? rep : 0;
    const uint32_t sela = ea ? 0x3254 : 0x3210, selb = eb ? 0x7610 : 0x3210;   // low / high lane from src
    const bool ea2 = ea == 2, eb2 = eb == 2;
    const uint32_t hcw = 0x00010001u * (uint32_t)((int)p.hcf + 1024);             // biased constant lanes
    // ... and at rows -1 / h: the band's first / last dx / dy row (steps 2 / nin-1) is
    // replaced by row 0 / h-1 (copy, Clamp / Mirror) or the constant row (Constant)
    const int fix_t = y0 == 0 && rep ? (rep == 2 ? 2 : 3) : -1;   // step of the fix
    const int fix_b = y0 + rows == g.h && rep ? nin - 1 : -1;
    const int mcol = active ? x : 0;
    const uint8_t *nrp = p.img + (ptrdiff_t)(y0 - 2) * g.pitch;
    auto issue = [&](int j, uint32_t slot) {
        const uint8_t *rp = nrp;
        if constexpr (CY) {
            const int yy = map_row1<true>(y0 - 2 + j, g.h, g.mode);
            if (yy < 0) {
                sts32(slot + 16 + loff, p.cword);
                if (lane == 0) sts32(slot + 12, p.cword);
                if (lane == 31) sts32(slot + 16 + FSTRIP, p.cword);
                return;
            }
            rp = p.img + (size_t)yy * g.pitch;
        }
        cpa4p(slot + 16 + loff, rp + mcol, active);
        cpa4p(slot + 12, rp + acol, aon);
        cpa4p(slot + bdst, rp + bcol, bon);
    };
#pragma unroll
    for (int j = 0; j < FLD; ++j) {
        issue(j, ring + j * FSLOT);
        nrp += g.pitch;
        cpa_commit();
    }
    // Laplace: box(i) = H(i) + Q(i-1) + Q(i-3) with Q(r) = H(r) + H(r-1), a ring of three Q
    // by step (pairs (H0,H2), (H1,H3)), bias 6400 per lane carried by the Q ring
    uint32_t lq[3][2] = {}, hp0 = 0, hp1 = 0;
    SobH sr[3];                              // Sobel horizontal parts, ring by step
    HRow hp, acc;                            // Harris: H(step-1) and H(step-2) + 2 H(step-1)
    const HRow hconst = {f2(p.c4, p.c4), f2(p.c4, p.c4), f2(p.c4, p.c4), f2(p.c4, p.c4), f2(p.c4, p.c4),
                         f2(p.c4, p.c4)};
    const float2 two = f2(2.f, 2.f);
    ptrdiff_t o4 = (ptrdiff_t)(y0 - 4) * g.out_pitch + x;   // output offset of row y0 + i - 4
#pragma unroll 1
    for (int i0 = 0; i0 < nin; i0 += 3) {
#pragma unroll
        for (int k = 0; k < 3; ++k) {
            const int i = i0 + k;
            if (i < nin) {
                cpa_wait<FLD - 1>();
                __syncwarp();
                const uint32_t sl = ring + (i & (FLR - 1)) * FSLOT + loff;
                const uint32_t W0 = lds32(sl + 16);
                const uint32_t L = __byte_perm(lds32(sl + 12), W0, sl_), R = __byte_perm(lds32(sl + 20), W0, sr_);
                const uint32_t F0 = __funnelshift_r(L, W0, 16), F1 = __funnelshift_r(W0, R, 16);
                const uint32_t Em2 = ev(F0), Om2 = od(F0), E0 = ev(W0), O0 = od(W0), E2 = ev(F1), O2 = od(F1);
                // ---- Laplace (a8): box of rows i-4..i, output row y0 + i - 4
                const uint32_t S = Om2 + E0 + O0 + E2;
                const uint32_t hn0 = S + Em2, hn1 = S + O2;
                const uint32_t box0 = hn0 + lq[(k + 2) % 3][0] + lq[k][0] + 0x19001900u;
                const uint32_t box1 = hn1 + lq[(k + 2) % 3][1] + lq[k][1] + 0x19001900u;
                lq[k][0] = hn0 + hp0;
                lq[k][1] = hn1 + hp1;
                hp0 = hn0;
                hp1 = hn1;
                // ---- Sobel horizontal parts of row i
                SobH &sh = sr[k];
                sh.sA = Em2 + 2u * Om2 + E0;
                sh.sE = Om2 + 2u * E0 + O0;
                sh.sO = E0 + 2u * O0 + E2;
                sh.sB = O0 + 2u * E2 + O2;
                sh.dA = E0 + 0x01000100u - Em2;
                sh.dE = O0 + 0x01000100u - Om2;
                sh.dO = E2 + 0x01000100u - E0;
                sh.dB = O2 + 0x01000100u - O0;
                if (i >= 4) {
                    const uint32_t c2 = lds32(ring + ((i - 2) & (FLR - 1)) * FSLOT + loff + 16);   // row i-2
                    uint32_t vE = box0 - 25u * ev(c2), vO = box1 - 25u * od(c2);
                    asm("max.u16x2 %0, %0, %1;" : "+r"(vE) : "r"(0x19001900u));
                    asm("min.u16x2 %0, %0, %1;" : "+r"(vE) : "r"(0x19FF19FFu));
                    asm("max.u16x2 %0, %0, %1;" : "+r"(vO) : "r"(0x19001900u));
                    asm("min.u16x2 %0, %0, %1;" : "+r"(vO) : "r"(0x19FF19FFu));
                    if (active) *reinterpret_cast<uint32_t *>(p.lap + o4) = __byte_perm(vE, vO, 0x6240);
                }
                if (i >= 2) {
                    // ---- dx / dy of row y0 + i - 3 (rows i-2, i-1, i), as exact floats
                    const SobH &a = sr[(k + 1) % 3], &b = sr[(k + 2) % 3];
                    const uint32_t dxA = a.dA + 2u * b.dA + sh.dA, dxE = a.dE + 2u * b.dE + sh.dE;
                    const uint32_t dxO = a.dO + 2u * b.dO + sh.dO, dxB = a.dB + 2u * b.dB + sh.dB;
                    const uint32_t dyA = sh.sA + 0x04000400u - a.sA, dyE = sh.sE + 0x04000400u - a.sE;
                    const uint32_t dyO = sh.sO + 0x04000400u - a.sO, dyB = sh.sB + 0x04000400u - a.sB;
                    // Harris reads the dx / dy images at remapped columns (edge lanes only):
                    // column -1 = the low lane of A, column w = the high lane of B, replaced
                    // by a byte permute (identity elsewhere) from column 0 / w-1 or the constant
                    const uint32_t xa = __byte_perm(dxA, ea2 ? hcw : dxE, sela), ya = __byte_perm(dyA, ea2 ? hcw : dyE, sela);
                    const uint32_t xb = __byte_perm(dxB, eb2 ? hcw : dxO, selb), yb = __byte_perm(dyB, eb2 ? hcw : dyO, selb);
                    const float2 xE = lanes_f(dxE, 1024.f), xO = lanes_f(dxO, 1024.f);
                    const float2 yE = lanes_f(dyE, 1024.f), yO = lanes_f(dyO, 1024.f);
                    const float2 xA = lanes_f(xa, 1024.f), xB = lanes_f(xb, 1024.f);
                    const float2 yA = lanes_f(ya, 1024.f), yB = lanes_f(yb, 1024.f);
                    HRow hn = har_hrow_f(xA, xE, xO, xB, yA, yE, yO, yB);
                    // ... and at remapped rows (the band's first / last dx / dy row)
                    if (i == fix_t) {
                        if (rep == 2) hn = hconst;
                        else hp = hn;   // step 3: row 0 also stands for row -1
                    }
                    if (i == fix_b) hn = rep == 2 ? hconst : hp;
                    // ---- magnitude (a9) and the optional dx / dy images of row y0 + i - 3
                    if (i >= 3 && i <= rows + 2) {
                        const ptrdiff_t o3 = o4 + g.out_pitch;
                        const float2 nE = fma2(xE, xE, mul2(yE, yE)), nO = fma2(xO, xO, mul2(yO, yO));
                        const uint32_t m0 = mag_bits(nE.x), m1 = mag_bits(nO.x), m2 = mag_bits(nE.y), m3 = mag_bits(nO.y);
                        const uint32_t mw = __byte_perm(__byte_perm(m0, m1, 0x0040), __byte_perm(m2, m3, 0x0040), 0x5410);
                        if (active) *reinterpret_cast<uint32_t *>(p.mag + o3) = mw;
                        if (DXY && active) {   // int16 = low half of the bits of v + 1.5 * 2^23
                            const float2 a2 = add2(xE, f2(12582912.f, 12582912.f)), b2 = add2(xO, f2(12582912.f, 12582912.f));
                            const float2 c2_ = add2(yE, f2(12582912.f, 12582912.f)), d2 = add2(yO, f2(12582912.f, 12582912.f));
                            *reinterpret_cast<uint2 *>(p.dx + o3) =
                                make_uint2(__byte_perm(__float_as_uint(a2.x), __float_as_uint(b2.x), 0x5410),
                                           __byte_perm(__float_as_uint(a2.y), __float_as_uint(b2.y), 0x5410));
                            *reinterpret_cast<uint2 *>(p.dy + o3) =
                                make_uint2(__byte_perm(__float_as_uint(c2_.x), __float_as_uint(d2.x), 0x5410),
                                           __byte_perm(__float_as_uint(c2_.y), __float_as_uint(d2.y), 0x5410));
                        }
                    }
                    if (i >= 4) {
                        // ---- Harris (a10) of row y0 + i - 4: dx / dy rows i-4 .. i-2 (steps)
                        // rows i-4 .. i-2 of dx / dy: acc (rows i-4, i-3) + the new row
                        const float2 sxxE = add2(acc.xxE, hn.xxE), sxxO = add2(acc.xxO, hn.xxO);
                        const float2 syyE = add2(acc.yyE, hn.yyE), syyO = add2(acc.yyO, hn.yyO);
                        const float2 sxyE = add2(acc.xyE, hn.xyE), sxyO = add2(acc.xyO, hn.xyO);
                        const uint32_t hw = harris4v(sxxE, syyE, sxyE, sxxO, syyO, sxyO, p.thr_f, p.thr_err, p.thr);
                        if (active) *reinterpret_cast<uint32_t *>(p.har + o4) = hw;
                    }
                    // vertical [1,2,1] as a running pair (two rows of state instead of three;
                    // integer sums < 2^24, exact in any order)
                    if (i > 2) {
                        acc.xxE = fma2(two, hn.xxE, hp.xxE); acc.xxO = fma2(two, hn.xxO, hp.xxO);
                        acc.yyE = fma2(two, hn.yyE, hp.yyE); acc.yyO = fma2(two, hn.yyO, hp.yyO);
                        acc.xyE = fma2(two, hn.xyE, hp.xyE); acc.xyO = fma2(two, hn.xyO, hp.xyO);
                    }
                    hp = hn;
                }
                o4 += g.out_pitch;
                if (i + FLD < nin) issue(i + FLD, ring + ((i + FLD) & (FLR - 1)) * FSLOT);
                nrp += g.pitch;
                cpa_commit();
            }
        }
    }
}

template <bool DXY>
__global__ void __launch_bounds__(NTB, FUSED_MINB) k_fused_band(const __grid_constant__ FusedBandParams p)
{
    __shared__ __align__(16) uint8_t rings[BW][FLR * FSLOT];
    asm volatile("griddepcontrol.wait;" ::: "memory");
    asm volatile("griddepcontrol.launch_dependents;");
    const BandGeom &g = p.g;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int gx = (int)blockIdx.x % g.ngx, band = (int)blockIdx.x / g.ngx;
    const int s = gx * BW + warp;
    if (s >= g.nstrip) return;
    int y0, y1;
    band_rows(band, g.nband, g.h, y0, y1);
    const bool cl = s < g.sx0, cr = s >= g.sx1, cy = band < g.by0 || band >= g.by1;
    const uint32_t ring = su32(rings[warp]);
    if (cy) fused_band_body<true, DXY>(p, ring, s * FSTRIP, y0, y1 - y0, lane, cl, cr);
    else fused_band_body<false, DXY>(p, ring, s * FSTRIP, y0, y1 - y0, lane, cl, cr);
}


// ------------------------------------------------------------------------------ Sobel
// Sobel dx, dy and magnitude (a9) on the same skeleton: 4 pixels per lane, rows y0-1 ..
// y0+rows streamed once; per row the horizontal parts s = a + 2b + c, d = c - a of the
// pairs E = (p0, p2), O = (p1, p3) on biased 16-bit lanes, two rows later dx = d + 2d + d,
// dy = s - s (bias 1024 per lane) -> exact floats -> magnitude (sqrt.approx, §7c) and the
// int16 images (low halves of v + 1.5 * 2^23).  Any subset of dx / dy / mag is written.
// Border handling is the staging's (rows mapped at copy time, edge lanes' halo bytes by
// selectors).  Bit-exact against the oracle.
struct SobBandParams {
    BandGeom g;
    const uint8_t *img;
    int16_t *dx, *dy;
    uint8_t *mag;
    uint32_t cword;
};

struct SobP { uint32_t sE, sO, dE, dO; };

template <int G, bool CY>
__device__ __forceinline__ void sob_band_body(const SobBandParams &p, uint32_t ring, int xs0, int y0, int rows,
                                              int lane, bool cl, bool cr)
{
    // G groups of 4 pixels per lane: strips of 128 G columns (BandShape<G>)
    using B = BandShape<G>;
    constexpr int LPX = B::LPX, STRIP = B::STRIP, SLOT = B::SLOT;
    const BandGeom &g = p.g;
    const int x = xs0 + LPX * lane;
    const bool active = !cr || x < g.w;
    const bool redge = cr && x + LPX == g.w;
    const int nin = rows + 2;   // >= 6
    const uint32_t loff = LPX * lane;
    int acol = xs0 - 4, bcol = xs0 + STRIP;
    uint32_t aon = lane == 0 && (!cl || g.mode == ISP_REPEAT), bdst = 16 + STRIP, bon = !cr && lane == 31;
    if (cl) acol = g.w - 4;
    if (redge && g.mode == ISP_REPEAT) { bon = 1; bcol = 0; bdst = 16 + LPX * (lane + 1); }
    uint32_t sl_ = 0x3210, sr_ = 0x3210;
    if (cl && lane == 0) sl_ = g.mode == ISP_CLAMP ? 0x4444 : g.mode == ISP_MIRROR ? 0x4500 : 0x3210;
    if (redge) sr_ = g.mode == ISP_CLAMP ? 0x7777 : g.mode == ISP_MIRROR ? 0x0067 : 0x3210;
    if (g.mode == ISP_CONSTANT) {
        for (int j = 0; j < LR; ++j) {
            if (cl && lane == 0) sts32(ring + j * SLOT + 12, p.cword);
            if (redge) sts32(ring + j * SLOT + 16 + LPX * (lane + 1), p.cword);
        }
    }
    const int mcol = active ? x : 0;
    const uint8_t *nrp = p.img + (ptrdiff_t)(y0 - 1) * g.pitch;
    auto issue = [&](int j, uint32_t slot) {
        const uint8_t *rp = nrp;
        if constexpr (CY) {
            const int yy = map_row1<true>(y0 - 1 + j, g.h, g.mode);
            if (yy < 0) {
#pragma unroll
                for (int q = 0; q < G; ++q) sts32(slot + 16 + loff + 4 * q, p.cword);
                if (lane == 0) sts32(slot + 12, p.cword);
                if (lane == 31) sts32(slot + 16 + STRIP, p.cword);
                return;
            }
            rp = p.img + (size_t)yy * g.pitch;
        }
        if constexpr (G == 1) cpa4p(slot + 16 + loff, rp + mcol, active);
        else cpa_own<G>(slot + 16 + loff, rp + mcol, active);
        cpa4p(slot + 12, rp + acol, aon);
        cpa4p(slot + bdst, rp + bcol, bon);
    };
#pragma unroll
    for (int j = 0; j < FLD; ++j) {
        issue(j, ring + j * SLOT);
        nrp += g.pitch;
        cpa_commit();
    }
    SobP sr[3][G];
    ptrdiff_t o2 = (ptrdiff_t)(y0 - 2) * g.out_pitch + x;   // output offset of row y0 + i - 2
    const float2 M = f2(12582912.f, 12582912.f);
#pragma unroll 1
    for (int i0 = 0; i0 < nin; i0 += 3) {
#pragma unroll
        for (int k = 0; k < 3; ++k) {
            const int i = i0 + k;
            if (i < nin) {
                cpa_wait<FLD - 1>();
                __syncwarp();
                const uint32_t sl = ring + (i & (LR - 1)) * SLOT + loff;
                uint32_t W[G + 2];   // [0] left halo word, [1..G] own, [G+1] right
                if constexpr (G == 1) W[1] = lds32(sl + 16);
                else lds_own<G>(sl + 16, *reinterpret_cast<uint32_t(*)[G]>(&W[1]));
                W[0] = __byte_perm(lds32(sl + 12), W[1], sl_);
                W[G + 1] = __byte_perm(lds32(sl + 16 + LPX), W[G], sr_);
#pragma unroll
                for (int q = 0; q < G; ++q) {
                    const uint32_t F0 = __funnelshift_r(W[q], W[q + 1], 16), F1 = __funnelshift_r(W[q + 1], W[q + 2], 16);
                    const uint32_t Om2 = od(F0), E0 = ev(W[q + 1]), O0 = od(W[q + 1]), E2 = ev(F1);
                    SobP &sh = sr[k][q];
                    sh.sE = Om2 + 2u * E0 + O0;
                    sh.sO = E0 + 2u * O0 + E2;
                    sh.dE = O0 + 0x01000100u - Om2;
                    sh.dO = E2 + 0x01000100u - E0;
                }
                if (i >= 2) {   // row y0 + i - 2 from rows i-2, i-1, i
                    uint32_t mw[G], dxw[2 * G], dyw[2 * G];
#pragma unroll
                    for (int q = 0; q < G; ++q) {
                        const SobP &a = sr[(k + 1) % 3][q], &b = sr[(k + 2) % 3][q], &sh = sr[k][q];
                        const uint32_t dxE = a.dE + 2u * b.dE + sh.dE, dxO = a.dO + 2u * b.dO + sh.dO;
                        const uint32_t dyE = sh.sE + 0x04000400u - a.sE, dyO = sh.sO + 0x04000400u - a.sO;
                        const float2 xE = lanes_f(dxE, 1024.f), xO = lanes_f(dxO, 1024.f);
                        const float2 yE = lanes_f(dyE, 1024.f), yO = lanes_f(dyO, 1024.f);
                        if (p.mag) {
                            const float2 nE = fma2(xE, xE, mul2(yE, yE)), nO = fma2(xO, xO, mul2(yO, yO));
                            const uint32_t m0 = mag_bits(nE.x), m1 = mag_bits(nO.x), m2 = mag_bits(nE.y),
                                           m3 = mag_bits(nO.y);
                            mw[q] = __byte_perm(__byte_perm(m0, m1, 0x0040), __byte_perm(m2, m3, 0x0040), 0x5410);
                        }
                        if (p.dx) {   // int16 = low half of the bits of v + 1.5 * 2^23
                            const float2 a2 = add2(xE, M), b2 = add2(xO, M);
                            dxw[2 * q] = __byte_perm(__float_as_uint(a2.x), __float_as_uint(b2.x), 0x5410);
                            dxw[2 * q + 1] = __byte_perm(__float_as_uint(a2.y), __float_as_uint(b2.y), 0x5410);
                        }
                        if (p.dy) {
                            const float2 a2 = add2(yE, M), b2 = add2(yO, M);
                            dyw[2 * q] = __byte_perm(__float_as_uint(a2.x), __float_as_uint(b2.x), 0x5410);
                            dyw[2 * q + 1] = __byte_perm(__float_as_uint(a2.y), __float_as_uint(b2.y), 0x5410);
                        }
                    }
                    if (active) {
                        if constexpr (G == 2) {
                            if (p.mag) *reinterpret_cast<uint2 *>(p.mag + o2) = make_uint2(mw[0], mw[1]);
                            if (p.dx) *reinterpret_cast<uint4 *>(p.dx + o2) = make_uint4(dxw[0], dxw[1], dxw[2], dxw[3]);
                            if (p.dy) *reinterpret_cast<uint4 *>(p.dy + o2) = make_uint4(dyw[0], dyw[1], dyw[2], dyw[3]);
                        } else {
                            if (p.mag) *reinterpret_cast<uint32_t *>(p.mag + o2) = mw[0];
                            if (p.dx) *reinterpret_cast<uint2 *>(p.dx + o2) = make_uint2(dxw[0], dxw[1]);
                            if (p.dy) *reinterpret_cast<uint2 *>(p.dy + o2) = make_uint2(dyw[0], dyw[1]);
                        }
                    }
                }
                o2 += g.out_pitch;
                if (i + FLD < nin) issue(i + FLD, ring + ((i + FLD) & (LR - 1)) * SLOT);
                nrp += g.pitch;
                cpa_commit();
            }
        }
    }
}

template <int G>
__global__ void __launch_bounds__(NTB, 8) k_sob_band(const __grid_constant__ SobBandParams p)
{
    __shared__ __align__(16) uint8_t rings[BW][LR * BandShape<G>::SLOT];
    asm volatile("griddepcontrol.wait;" ::: "memory");
    asm volatile("griddepcontrol.launch_dependents;");
    const BandGeom &g = p.g;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int gx = (int)blockIdx.x % g.ngx, band = (int)blockIdx.x / g.ngx;
    const int s = gx * BW + warp;
    if (s >= g.nstrip) return;
    int y0, y1;
    band_rows(band, g.nband, g.h, y0, y1);
    const bool cl = s < g.sx0, cr = s >= g.sx1, cy = band < g.by0 || band >= g.by1;
    const uint32_t ring = su32(rings[warp]);
    if (cy) sob_band_body<G, true>(p, ring, s * BandShape<G>::STRIP, y0, y1 - y0, lane, cl, cr);
    else sob_band_body<G, false>(p, ring, s * BandShape<G>::STRIP, y0, y1 - y0, lane, cl, cr);
}

// pixel groups of 4 per lane of the Sobel band launch: 2 unless ISP_SOBEL_G=1
int sobel_g()
{
    const char *e = getenv("ISP_SOBEL_G");
    return e && atoi(e) == 1 ? 1 : 2;
}
const void *sob_band_fn(int gq) { return gq == 1 ? (const void *)k_sob_band<1> : (const void *)k_sob_band<2>; }
int sob_blocks_per_sm(int gq)
{
    static int nb[3] = {-1, -1, -1};
    if (nb[gq] < 0) {
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb[gq], sob_band_fn(gq), NTB, 0) != cudaSuccess) {
            cudaGetLastError();
            nb[gq] = 0;
        }
    }
    return nb[gq];
}

// ------------------------------------------------------------------------------ separable u8
// Separable u8 masks with non-negative integer weights whose products sum to at most the
// divisor d = 2^s <= 256 (the binomial Gaussians of a7: 3x3 / 16, 5x5 / 256): every
// horizontal sum and the 2-D sum fit a 16-bit lane, so the Laplace skeleton carries them
// as pair lanes (E = pixels (0,2), O = (1,3)).  Horizontal K-tap sums by DP4A on byte
// windows (5 taps: two DP4A, the second with weights (0,0,0,r4) on the next window),
// vertical K-tap weighted sums over a register ring of K rows, then round-half-up by
// adding d/2 and taking bits [s, s+8) of each lane (exact: U8Round with a power-of-two
// divisor; no saturation is needed since the result is <= 255).
struct SepU8BandParams {
    BandGeom g;
    const uint8_t *img;
    uint8_t *out;
    uint32_t cword;
    uint32_t r03, r4w;   // DP4A weight words: (r0, r1, r2, r3) and (0, 0, 0, r4) (K = 3: (r0, r1, r2, 0), 0)
    int col[5];
    int shift;           // s: d = 2^s
};

template <int NW, int K, bool CY>
__device__ __forceinline__ void sepu8_band_body(const SepU8BandParams &p, uint32_t ring, int xs0, int y0, int rows,
                                                int lane, bool cl, bool cr)
{
    using B = BandShape<NW>;
    constexpr int LPX = B::LPX, STRIP = B::STRIP, SLOT = B::SLOT, HY = K / 2;
    const BandGeom &g = p.g;
    const int x = xs0 + LPX * lane;
    const bool active = !cr || x < g.w;
    const bool redge = cr && x + LPX == g.w;
    const int nin = rows + 2 * HY;
    const uint32_t loff = LPX * lane;
    int acol = xs0 - 4, bcol = xs0 + STRIP;
    uint32_t aon = lane == 0 && (!cl || g.mode == ISP_REPEAT), bdst = 16 + STRIP, bon = !cr && lane == 31;
    if (cl) acol = g.w - 4;
    if (redge && g.mode == ISP_REPEAT) { bon = 1; bcol = 0; bdst = 16 + LPX * (lane + 1); }
    uint32_t sl_ = 0x3210, sr_ = 0x3210;
    if (cl && lane == 0) sl_ = g.mode == ISP_CLAMP ? 0x4444 : g.mode == ISP_MIRROR ? 0x4500 : 0x3210;
    if (redge) sr_ = g.mode == ISP_CLAMP ? 0x7777 : g.mode == ISP_MIRROR ? 0x0067 : 0x3210;
    if (g.mode == ISP_CONSTANT) {
        for (int j = 0; j < LR; ++j) {
            if (cl && lane == 0) sts32(ring + j * SLOT + 12, p.cword);
            if (redge) sts32(ring + j * SLOT + 16 + LPX * (lane + 1), p.cword);
        }
    }
    const int mcol = active ? x : 0;
    const uint8_t *nrp = p.img + (ptrdiff_t)(y0 - HY) * g.pitch;
    auto issue = [&](int j, uint32_t slot) {
        const uint8_t *rp = nrp;
        if constexpr (CY) {
            const int yy = map_row1<true>(y0 - HY + j, g.h, g.mode);
            if (yy < 0) {
#pragma unroll
                for (int q = 0; q < NW; ++q) sts32(slot + 16 + loff + 4 * q, p.cword);
                if (lane == 0) sts32(slot + 12, p.cword);
                if (lane == 31) sts32(slot + 16 + STRIP, p.cword);
                return;
            }
            rp = p.img + (size_t)yy * g.pitch;
        }
        cpa_own<NW>(slot + 16 + loff, rp + mcol, active);
        cpa4p(slot + 12, rp + acol, aon);
        cpa4p(slot + bdst, rp + bcol, bon);
    };
#pragma unroll
    for (int j = 0; j < LD; ++j) {
        issue(j, ring + j * SLOT);
        nrp += g.pitch;
        cpa_commit();
    }
    const uint32_t halfw = 0x00010001u * (uint32_t)((1 << p.shift) >> 1);
    uint32_t hr[K][2 * NW];   // horizontal sums of the last K rows as pair lanes (E0, O0, E1, O1)
    uint8_t *orow = p.out + (ptrdiff_t)(y0 - (K - 1)) * g.out_pitch + x;
#pragma unroll 1
    for (int i0 = 0; i0 < nin; i0 += K) {
#pragma unroll
        for (int k = 0; k < K; ++k) {
            const int i = i0 + k;
            if (i < nin) {
                cpa_wait<LD - 1>();
                __syncwarp();
                const uint32_t sl = ring + (i & (LR - 1)) * SLOT + loff;
                uint32_t W[NW + 2];
                lds_own<NW>(sl + 16, *reinterpret_cast<uint32_t(*)[NW]>(&W[1]));
                W[0] = __byte_perm(lds32(sl + 12), W[1], sl_);
                W[NW + 1] = __byte_perm(lds32(sl + 16 + LPX), W[NW], sr_);
                // byte windows F[j] = bytes j-2 .. j+1 relative to the lane's pixel 0, j = 0..4 NW
                constexpr int NPX = 4 * NW;
                uint32_t F[NPX + 1];
#pragma unroll
                for (int j = 0; j <= NPX; ++j) {
                    const int q = (j + 2) >> 2, sh = (j + 2) & 3;   // window starts in word q-1 ... of W (offset -4)
                    F[j] = sh == 0 ? W[q] : __funnelshift_r(W[q], W[q + 1], 8 * sh);
                }
                uint32_t H[NPX];
#pragma unroll
                for (int px = 0; px < NPX; ++px) {
                    if constexpr (K == 5) H[px] = __dp4a(F[px + 1], p.r4w, __dp4a(F[px], p.r03, 0u));   // bytes px-2..px+2
                    else H[px] = __dp4a(F[px + 1], p.r03, 0u);                                        // bytes px-1..px+1
                }
                uint32_t(&hn)[2 * NW] = hr[k];
#pragma unroll
                for (int q = 0; q < NW; ++q) {
                    hn[2 * q] = H[4 * q + 2] * 65536u + H[4 * q];
                    hn[2 * q + 1] = H[4 * q + 3] * 65536u + H[4 * q + 1];
                }
                if (i >= K - 1 && active) {
                    // output row y0 + i - (K-1): rows i-K+1 .. i = ring slots (k+1+j) % K
                    uint32_t v[2 * NW];
#pragma unroll
                    for (int q = 0; q < 2 * NW; ++q) {
                        uint32_t a = halfw;
#pragma unroll
                        for (int j = 0; j < K; ++j) a += (uint32_t)p.col[j] * hr[(k + 1 + j) % K][q];
                        v[q] = (a >> p.shift) & 0x00FF00FFu;
                    }
                    if constexpr (NW == 4)
                        *reinterpret_cast<uint4 *>(orow) =
                            make_uint4(__byte_perm(v[0], v[1], 0x6240), __byte_perm(v[2], v[3], 0x6240),
                                       __byte_perm(v[4], v[5], 0x6240), __byte_perm(v[6], v[7], 0x6240));
                    else
                        *reinterpret_cast<uint2 *>(orow) =
                            make_uint2(__byte_perm(v[0], v[1], 0x6240), __byte_perm(v[2], v[3], 0x6240));
                }
                orow += g.out_pitch;
                if (i + LD < nin) issue(i + LD, ring + ((i + LD) & (LR - 1)) * SLOT);
                nrp += g.pitch;
                cpa_commit();
            }
        }
    }
}

template <int NW, int K>
__global__ void __launch_bounds__(NTB, NW == 2 ? 8 : 5) k_sepu8_band(const __grid_constant__ SepU8BandParams p)
{
    __shared__ __align__(16) uint8_t rings[BW][LR * BandShape<NW>::SLOT];
    asm volatile("griddepcontrol.wait;" ::: "memory");
    asm volatile("griddepcontrol.launch_dependents;");
    const BandGeom &g = p.g;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int gx = (int)blockIdx.x % g.ngx, band = (int)blockIdx.x / g.ngx;
    const int s = gx * BW + warp;
    if (s >= g.nstrip) return;
    int y0, y1;
    band_rows(band, g.nband, g.h, y0, y1);
    const bool cl = s < g.sx0, cr = s >= g.sx1, cy = band < g.by0 || band >= g.by1;
    const uint32_t ring = su32(rings[warp]);
    if (cy) sepu8_band_body<NW, K, true>(p, ring, s * BandShape<NW>::STRIP, y0, y1 - y0, lane, cl, cr);
    else sepu8_band_body<NW, K, false>(p, ring, s * BandShape<NW>::STRIP, y0, y1 - y0, lane, cl, cr);
}

// words (4 pixels) per lane of the separable u8 band launch: 4 unless ISP_SEPU8_NW=2
int sepu8_nw()
{
    const char *e = getenv("ISP_SEPU8_NW");
    return e && atoi(e) == 2 ? 2 : 4;
}
const void *sepu8_fn(int nw, int k)
{
    if (nw == 2) return k == 5 ? (const void *)k_sepu8_band<2, 5> : (const void *)k_sepu8_band<2, 3>;
    return k == 5 ? (const void *)k_sepu8_band<4, 5> : (const void *)k_sepu8_band<4, 3>;
}

int sepu8_blocks_per_sm(int k)
{
    static int nb[2][2] = {{-1, -1}, {-1, -1}};
    const int nw = sepu8_nw();
    int &v = nb[nw == 4][k == 5];
    if (v < 0) {
        const void *fn = sepu8_fn(nw, k);
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&v, fn, NTB, 0) != cudaSuccess) {
            cudaGetLastError();
            v = 0;
        }
    }
    return v;
}

// Words per lane of the Laplace band launch: 4 (16 pixels) unless ISP_BAND_NW=2
int band_nw()
{
    const char *e = getenv("ISP_BAND_NW");
    return e && atoi(e) == 2 ? 2 : 4;
}

const void *lap_band_fn(int nw) { return nw == 2 ? (const void *)k_lap_band<2> : (const void *)k_lap_band<4>; }

// resident CTAs per SM: which = 2 / 4 (Laplace, NW words per lane), 1 (Harris), 3 (fused cfg3),
// 0 (Sobel)
int band_blocks_per_sm(int which)
{
    static int nb[5] = {-1, -1, -1, -1, -1};
    if (nb[which] < 0) {
        const void *fn = which == 1   ? har_band_fn(harris_g())
                         : which == 3 ? (const void *)k_fused_band<false>
                         : which == 0 ? sob_band_fn(sobel_g())
                                      : lap_band_fn(which);
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb[which], fn, NTB, 0) != cudaSuccess) {
            cudaGetLastError();
            nb[which] = 0;
        }
    }
    return nb[which];
}

}  // namespace

// Eligibility of the band kernels: 16-pixel lane granules (w % 16 == 0; 8 with
// ISP_BAND_NW=2), rows aligned to the granule in and out (cp.async / vector stores), and
// h >= 8 so that every overshoot needs one reflection.
bool ispi_band_ok(const void *in, int w, int h, int pitch, const void *out, int out_pitch)
{
    const int v = 4 * band_nw();
    auto al = [](const void *q, long long pb, int a) { return q && ((uintptr_t)q % a) == 0 && (pb % a) == 0; };
    return al(in, pitch, v) && al(out, out_pitch, v) && w % v == 0 && w >= 2 * v && h >= 8;
}

// Strip width and band height of the Laplace band launch (the model's tile shape, Eq. 2 / 10).
void ispi_band_shape(int w, int h, int *tw, int *th)
{
    const int nw = band_nw();
    const BandGeom g = band_geom(w, h, w, w, ISP_CLAMP, 2, 128 * nw, band_blocks_per_sm(nw), bands_hint());
    *tw = 128 * nw;
    *th = (h + g.nband - 1) / g.nband;
}

int ispi_band_blocks_per_sm(int which)
{
    return which == 1 ? har_blocks_per_sm(harris_g()) : which == 2 ? sob_blocks_per_sm(sobel_g())
                                                              : band_blocks_per_sm(band_nw());
}

cudaError_t ispi_laplace_band(const uint8_t *img, int w, int h, int pitch, int mode, int cval, uint8_t *out,
                              int out_pitch, cudaStream_t st, int bounds[4])
{
    const int nw = band_nw();
    LapBandParams p{};
    p.g = band_geom(w, h, pitch, out_pitch, mode, 2, 128 * nw, band_blocks_per_sm(nw), bands_hint());
    p.img = img;
    p.out = out;
    p.cword = 0x01010101u * (uint32_t)(cval & 0xff);
    bounds[0] = p.g.sx0; bounds[1] = std::max(p.g.sx0, p.g.sx1); bounds[2] = p.g.by0; bounds[3] = p.g.by1;
    return launch_band(lap_band_fn(nw), &p, p.g.ngx * p.g.nband, st);
}

// Harris band kernel: 4 G-pixel lane granules of int16 (8 G-byte aligned rows), 4 G-byte
// aligned output rows, h >= 8.
bool ispi_band_harris_ok(const void *dx, const void *dy, int w, int h, int pitch, const void *out, int out_pitch)
{
    auto al = [](const void *q, long long pb, int a) { return q && ((uintptr_t)q % a) == 0 && (pb % a) == 0; };
    const int gq = harris_g();
    return al(dx, 2LL * pitch, 8 * gq) && al(dy, 2LL * pitch, 8 * gq) && al(out, out_pitch, 4 * gq) &&
           w % (4 * gq) == 0 && w >= 8 * gq && h >= 8;
}

void ispi_band_harris_shape(int w, int h, int *tw, int *th)
{
    const int gq = harris_g();
    const BandGeom g = band_geom(w, h, w, w, ISP_CLAMP, 1, 128 * gq, har_blocks_per_sm(gq), bands_hint());
    *tw = 128 * gq;
    *th = (h + g.nband - 1) / g.nband;
}

cudaError_t ispi_harris_band(const int16_t *dx, const int16_t *dy, int w, int h, int pitch, int mode, int cval,
                             long long thr, uint8_t *out, int out_pitch, cudaStream_t st, int bounds[4])
{
    HarBandParams p{};
    const int gq = harris_g();
    p.g = band_geom(w, h, pitch, out_pitch, mode, 1, 128 * gq, har_blocks_per_sm(gq), bands_hint());
    p.dx = dx;
    p.dy = dy;
    p.out = out;
    p.cword = 0x00010001u * (uint32_t)(uint16_t)(int16_t)cval;
    p.thr = (double)std::max(-9007199254740992ll, std::min(9007199254740992ll, thr));
    p.thr_f = (float)p.thr;
    p.thr_err = thr_bound(p.thr_f);
    bounds[0] = p.g.sx0; bounds[1] = std::max(p.g.sx0, p.g.sx1); bounds[2] = p.g.by0; bounds[3] = p.g.by1;
    return launch_band(har_band_fn(gq), &p, p.g.ngx * p.g.nband, st);
}

// Fused cfg3 band kernel: 4-pixel lane granules, 4-byte aligned rows in and out (8-byte for
// the optional dx / dy), h >= 8.
bool ispi_band_fused_ok(const void *img, int w, int h, int pitch, const void *mag, const void *lap, const void *har,
                        const void *dx, const void *dy, int out_pitch)
{
    auto al = [](const void *q, long long pb, int a) { return ((uintptr_t)q % a) == 0 && (pb % a) == 0; };
    return al(img, pitch, 4) && al(mag, out_pitch, 4) && al(lap, out_pitch, 4) && al(har, out_pitch, 4) &&
           (!dx || al(dx, 2LL * out_pitch, 8)) && (!dy || al(dy, 2LL * out_pitch, 8)) && (!dx == !dy) && w % 4 == 0 &&
           w >= 8 && h >= 8;
}

cudaError_t ispi_fused_band(const uint8_t *img, int w, int h, int pitch, int mode, int cval, int hcval, long long thr,
                            int16_t *dx, int16_t *dy, uint8_t *mag, uint8_t *lap, uint8_t *har, int out_pitch,
                            cudaStream_t st)
{
    FusedBandParams p{};
    p.g = band_geom(w, h, pitch, out_pitch, mode, 2, FSTRIP, band_blocks_per_sm(3), bands_hint());
    p.img = img;
    p.mag = mag; p.lap = lap; p.har = har; p.dx = dx; p.dy = dy;
    p.cword = 0x01010101u * (uint32_t)(cval & 0xff);
    p.hcf = (float)hcval;
    p.c4 = 4.0f * (float)hcval * (float)hcval;
    p.thr = (double)std::max(-9007199254740992ll, std::min(9007199254740992ll, thr));
    p.thr_f = (float)p.thr;
    p.thr_err = thr_bound(p.thr_f);
    return launch_band(p.dx ? (const void *)k_fused_band<true> : (const void *)k_fused_band<false>, &p,
                       p.g.ngx * p.g.nband, st);
}

// Sobel band kernel: 4 G-pixel lane granules, 4 G-byte aligned input and mag rows, 8 G-byte
// aligned dx / dy rows, h >= 8.
bool ispi_band_sobel_ok(const void *img, int w, int h, int pitch, const void *dx, const void *dy, const void *mag,
                        int out_pitch)
{
    auto al = [](const void *q, long long pb, int a) { return ((uintptr_t)q % a) == 0 && (pb % a) == 0; };
    const int gq = sobel_g(), v = 4 * gq;
    return al(img, pitch, v) && (!mag || al(mag, out_pitch, v)) && (!dx || al(dx, 2LL * out_pitch, 2 * v)) &&
           (!dy || al(dy, 2LL * out_pitch, 2 * v)) && w % v == 0 && w >= 2 * v && h >= 8;
}

void ispi_band_sobel_shape(int w, int h, int *tw, int *th)
{
    const int gq = sobel_g();
    const BandGeom g = band_geom(w, h, w, w, ISP_CLAMP, 1, 128 * gq, sob_blocks_per_sm(gq), bands_hint());
    *tw = 128 * gq;
    *th = (h + g.nband - 1) / g.nband;
}

cudaError_t ispi_sobel_band(const uint8_t *img, int w, int h, int pitch, int mode, int cval, int16_t *dx, int16_t *dy,
                            uint8_t *mag, int out_pitch, cudaStream_t st, int bounds[4])
{
    SobBandParams p{};
    const int gq = sobel_g();
    p.g = band_geom(w, h, pitch, out_pitch, mode, 1, 128 * gq, sob_blocks_per_sm(gq), bands_hint());
    p.img = img;
    p.dx = dx; p.dy = dy; p.mag = mag;
    p.cword = 0x01010101u * (uint32_t)(cval & 0xff);
    bounds[0] = p.g.sx0; bounds[1] = std::max(p.g.sx0, p.g.sx1); bounds[2] = p.g.by0; bounds[3] = p.g.by1;
    return launch_band(sob_band_fn(gq), &p, p.g.ngx * p.g.nband, st);
}

// Separable u8 band kernel eligibility: K = 3 / 5, non-negative weights, divisor 2^s <= 256
// with sum(row) * sum(col) <= divisor (16-bit lanes, no saturation), 8-pixel lane granules,
// 8-byte aligned rows, h >= 8.
bool ispi_sepu8_band_ok(const void *img, int w, int h, int pitch, const void *out, int out_pitch, int k,
                        const int *row, const int *col, int divisor)
{
    auto al = [](const void *q, long long pb, int a) { return ((uintptr_t)q % a) == 0 && (pb % a) == 0; };
    if ((k != 3 && k != 5) || divisor <= 0 || divisor > 256 || (divisor & (divisor - 1)) != 0) return false;
    long long sr = 0, sc = 0;
    for (int i = 0; i < k; ++i) {
        if (row[i] < 0 || col[i] < 0 || row[i] > 255) return false;
        sr += row[i];
        sc += col[i];
    }
    const int v = 4 * sepu8_nw();
    return sr * sc <= divisor && al(img, pitch, v) && al(out, out_pitch, v) && w % v == 0 && w >= 2 * v && h >= 8;
}

void ispi_sepu8_band_shape(int w, int h, int k, int *tw, int *th)
{
    const int strip = 128 * sepu8_nw();
    const BandGeom g = band_geom(w, h, w, w, ISP_CLAMP, k / 2, strip, sepu8_blocks_per_sm(k), bands_hint());
    *tw = strip;
    *th = (h + g.nband - 1) / g.nband;
}

int ispi_sepu8_band_blocks_per_sm(int k) { return sepu8_blocks_per_sm(k); }

cudaError_t ispi_sepu8_band(const uint8_t *img, int w, int h, int pitch, int k, const int *row, const int *col,
                            int divisor, int mode, int cval, uint8_t *out, int out_pitch, cudaStream_t st, int bounds[4])
{
    SepU8BandParams p{};
    const int nw = sepu8_nw();
    p.g = band_geom(w, h, pitch, out_pitch, mode, k / 2, 128 * nw, sepu8_blocks_per_sm(k), bands_hint());
    p.img = img;
    p.out = out;
    p.cword = 0x01010101u * (uint32_t)(cval & 0xff);
    if (k == 5) {
        p.r03 = (uint32_t)row[0] | (uint32_t)row[1] << 8 | (uint32_t)row[2] << 16 | (uint32_t)row[3] << 24;
        p.r4w = (uint32_t)row[4] << 24;
    } else {
        p.r03 = (uint32_t)row[0] | (uint32_t)row[1] << 8 | (uint32_t)row[2] << 16;
        p.r4w = 0;
    }
    for (int j = 0; j < k; ++j) p.col[j] = col[j];
    int s = 0;
    while ((1 << s) < divisor) ++s;
    p.shift = s;
    bounds[0] = p.g.sx0; bounds[1] = std::max(p.g.sx0, p.g.sx1); bounds[2] = p.g.by0; bounds[3] = p.g.by1;
    return launch_band(sepu8_fn(nw, k), &p, p.g.ngx * p.g.nband, st);
}
