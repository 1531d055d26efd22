// band_f32.cu -- warp-strip streaming ISP kernel for separable f32 masks (a7: the cfg2 /
// cfg5 Gaussians): the ISP_TMA / ISP_AUTO kernel of isp_filter for whole images (the
// TMA-staged k_staged of isp_staged.cuh remains for strips and with ISP_F32_STAGED=1);
// 4096^2 5x5 28.8 -> 27.1 us, 16384^2 7x7 420 -> 379 us.
//
// Partition as in band_u8.cu (band_common.cuh): warp strips of 32 lanes x 4 pixels (one
// float4 per lane, 128 columns) by balanced row bands; each warp streams its rows through
// its own shared-memory ring with cp.async (16 bytes per lane, the strip's 16-byte halo
// vectors by lanes 0 and 31), LD rows in flight.  Regions (Listing 3 per warp, template
// bodies): T / B warps map their out-of-image rows through the pattern at copy time
// (Constant: the staged row is C); L / R warps rebuild the halo columns beyond the edge in
// registers (Clamp / Mirror), pre-store C (Constant) or copy the wrapped vector (Repeat);
// Body warps run no check.  The arithmetic is OpSepF32's (isp_ops.cuh) in the same order --
// the row pass as FP32x2 FMA chains over the taps, the column pass into MH accumulators in
// row order -- so results are bitwise those of every other variant.
#include <cuda_runtime.h>
#include <stdint.h>

#include <algorithm>
#include <cstdlib>
#include <cstring>

#include "../../include/isp.h"
#include "internal.h"
#include "band_common.cuh"

namespace {

constexpr int SPX = 4, SSTRIP = 32 * SPX;          // pixels per lane / columns per warp
constexpr int SSLOT = 16 + 4 * SSTRIP + 16;        // bytes: left halo vector, strip, right halo vector
#ifndef BAND_F32_D
#define BAND_F32_D 3   // 3 rows in flight per warp measured best (cfg2 / cfg5)
#endif
constexpr int SLD = BAND_F32_D;
#ifndef BAND_F32_HALF
#define BAND_F32_HALF 2   // halo columns loaded as half vectors up to this reach
#endif
static_assert(LR >= SLD + 1, "ring too small");

// Output rows [oy0, oy0 + nrows) of an image of height g.h (whole image: 0, h); strips of
// the multi-GPU path (readings A30 / A32): an edge that is not an image edge
// (t_real / b_real = 0) is a strip edge -- its rows are in the buffer (NCCL halo exchange)
// or, with peer != 0, in the neighbour strips' buffers peer_lo / peer_hi (global-row
// addressed, rows < own_y0 / >= own_y1).
struct SepBandRows {
    int oy0, nrows, t_real, b_real, peer, own_y0, own_y1;
    const float *peer_lo, *peer_hi;
};

struct SepBandParams {
    BandGeom g;
    SepBandRows rr;
    const float *img;
    float *out;
    float cval;
    float row[7], col[7];
};

__device__ __forceinline__ void fma2s(float &a0, float &a1, float c, float b0, float b1)
{
    const float2 r = __ffma2_rn(make_float2(c, c), make_float2(b0, b1), make_float2(a0, a1));
    a0 = r.x;
    a1 = r.y;
}
__device__ __forceinline__ void mul2s(float &a0, float &a1, float c, float b0, float b1)
{
    const float2 r = __fmul2_rn(make_float2(c, c), make_float2(b0, b1));
    a0 = r.x;
    a1 = r.y;
}
__device__ __forceinline__ void cpa16p(uint32_t dst, const void *src, uint32_t on)
{
    asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %2, 0;\n\t@q cp.async.cg.shared.global [%0], [%1], 16;\n\t}" ::"r"(dst),
                 "l"(src), "r"(on)
                 : "memory");
}
__device__ __forceinline__ float4 lds128f(uint32_t a)
{
    float4 v;
    asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "r"(a)
                 : "memory");
    return v;
}
__device__ __forceinline__ float2 lds64f(uint32_t a)
{
    float2 v;
    asm volatile("ld.shared.v2.f32 {%0, %1}, [%2];" : "=f"(v.x), "=f"(v.y) : "r"(a) : "memory");
    return v;
}
__device__ __forceinline__ void sts128f(uint32_t a, float v)
{
    asm volatile("st.shared.v4.f32 [%0], {%1, %1, %1, %1};" ::"r"(a), "f"(v) : "memory");
}

template <int K, bool CL, bool CR, bool CY>
__device__ __forceinline__ void sep_band_body(const SepBandParams &p, uint32_t ring, int xs0, int y0, int rows, int lane)
{
    constexpr int HX = K / 2, SEGW = SPX + 2 * HX;
    const BandGeom &g = p.g;
    const int x = xs0 + SPX * lane;
    const bool active = !CR || x < g.w;
    const bool redge = CR && x + SPX == g.w;
    const int nin = rows + 2 * HX;
    const uint32_t loff = 16 * lane;
    // copies per row: the lane's vector (none past the image); A: lane 0 the strip's left
    // halo vector (L, Repeat: the wrapped columns w-4..w-1); B: lane 31 the right one, or
    // (R, Repeat) the image's last lane the wrapped columns 0..3 into its neighbour's place
    int acol = xs0 - 4, bcol = xs0 + SSTRIP;
    uint32_t aon = lane == 0 && (!CL || g.mode == ISP_REPEAT), bdst = 16 + 4 * SSTRIP, bon = !CR && lane == 31;
    if (CL) acol = g.w - 4;
    if (redge && g.mode == ISP_REPEAT) { bon = 1; bcol = 0; bdst = 16 + 16 * (lane + 1); }
    if (g.mode == ISP_CONSTANT) {   // the halo positions no copy writes hold C in every slot
        for (int j = 0; j < LR; ++j) {
            if (CL && lane == 0) sts128f(ring + j * SSLOT, p.cval);
            if (redge) sts128f(ring + j * SSLOT + 16 + 16 * (lane + 1), p.cval);
        }
    }
    const int mcol = active ? x : 0;
    const float *nrp = p.img + (ptrdiff_t)(y0 - HX) * g.pitch;
    auto issue = [&](int j, uint32_t slot) {
        const float *rp = nrp;
        if constexpr (CY) {   // T / B: image edges through the pattern, strip edges by buffer
            const int y = y0 - HX + j;
            const bool out_img = (p.rr.t_real && y < 0) || (p.rr.b_real && y >= g.h);
            const int yy = out_img ? map_row1<true>(y, g.h, g.mode) : y;
            if (out_img && yy < 0) {   // Constant: the staged row is C
                sts128f(slot + 16 + loff, p.cval);
                if (lane == 0) sts128f(slot, p.cval);
                if (lane == 31) sts128f(slot + 16 + 4 * SSTRIP, p.cval);
                return;
            }
            const float *base = p.img;
            if (p.rr.peer) {
                if (yy < p.rr.own_y0) base = p.rr.peer_lo;
                else if (yy >= p.rr.own_y1) base = p.rr.peer_hi;
            }
            rp = base + (ptrdiff_t)yy * g.pitch;
        }
        cpa16p(slot + 16 + loff, rp + mcol, active);
        cpa16p(slot, rp + acol, aon);
        cpa16p(slot + bdst, rp + bcol, bon);
    };
#pragma unroll
    for (int j = 0; j < SLD; ++j) {
        issue(j, ring + j * SSLOT);
        nrp += g.pitch;
        cpa_commit();
    }
    float acc[K][SPX];
    float *orow = p.out + (ptrdiff_t)(y0 - p.rr.oy0 - (K - 1)) * g.out_pitch + x;   // output o = r - (K-1)
#pragma unroll 1
    for (int r0 = 0; r0 < nin; r0 += K) {
#pragma unroll
        for (int k = 0; k < K; ++k) {
            const int r = r0 + k;
            if (r < nin) {
                cpa_wait<SLD - 1>();
                __syncwarp();
                const uint32_t sl = ring + (r & (LR - 1)) * SSLOT + loff;
                const float4 o = lds128f(sl + 16);
                // halo columns: the neighbours' nearest HX values (half vectors for HX <= 2)
                float4 L, R;
                if constexpr (HX <= BAND_F32_HALF) {
                    const float2 l2 = lds64f(sl + 8), r2 = lds64f(sl + 32);
                    L = make_float4(0.f, 0.f, l2.x, l2.y);
                    R = make_float4(r2.x, r2.y, 0.f, 0.f);
                } else {
                    L = lds128f(sl);
                    R = lds128f(sl + 32);
                }
                if constexpr (CL) {   // columns -4..-1 through Clamp / Mirror (lane 0)
                    if (lane == 0 && g.mode == ISP_CLAMP) L = make_float4(o.x, o.x, o.x, o.x);
                    if (lane == 0 && g.mode == ISP_MIRROR) L = make_float4(o.w, o.z, o.y, o.x);
                }
                if constexpr (CR) {   // columns w..w+3 (the image's last lane)
                    if (redge && g.mode == ISP_CLAMP) R = make_float4(o.w, o.w, o.w, o.w);
                    if (redge && g.mode == ISP_MIRROR) R = make_float4(o.w, o.z, o.y, o.x);
                }
                const float lv[4] = {L.x, L.y, L.z, L.w}, rv[4] = {R.x, R.y, R.z, R.w};
                float seg[SEGW];
#pragma unroll
                for (int q = 0; q < HX; ++q) {
                    seg[q] = lv[4 - HX + q];
                    seg[HX + SPX + q] = rv[q];
                }
                seg[HX] = o.x; seg[HX + 1] = o.y; seg[HX + 2] = o.z; seg[HX + 3] = o.w;
                // row pass (OpSepF32::hrow order)
                float hs[SPX];
#pragma unroll
                for (int e = 0; e < SPX; e += 2) {
                    float t0, t1;
                    mul2s(t0, t1, p.row[0], seg[e], seg[e + 1]);
#pragma unroll
                    for (int i = 1; i < K; ++i) fma2s(t0, t1, p.row[i], seg[e + i], seg[e + i + 1]);
                    hs[e] = t0;
                    hs[e + 1] = t1;
                }
                // column pass (OpSepF32::vacc order): tap 0 starts the row's accumulator
#pragma unroll
                for (int e = 0; e < SPX; e += 2) mul2s(acc[k][e], acc[k][e + 1], p.col[0], hs[e], hs[e + 1]);
#pragma unroll
                for (int j = 1; j < K; ++j)
#pragma unroll
                    for (int e = 0; e < SPX; e += 2)
                        fma2s(acc[(k - j + K) % K][e], acc[(k - j + K) % K][e + 1], p.col[j], hs[e], hs[e + 1]);
                if (r >= K - 1 && active) {
                    const float(&a)[SPX] = acc[(k + 1) % K];
                    *reinterpret_cast<float4 *>(orow) = make_float4(a[0], a[1], a[2], a[3]);
                }
                orow += g.out_pitch;
                if (r + SLD < nin) issue(r + SLD, ring + ((r + SLD) & (LR - 1)) * SSLOT);
                nrp += g.pitch;
                cpa_commit();
            }
        }
    }
}

#ifndef BAND_F32_MINB
#define BAND_F32_MINB 6
#endif
template <int K>
__global__ void __launch_bounds__(NTB, BAND_F32_MINB) k_sep_band(const __grid_constant__ SepBandParams p)
{
    __shared__ __align__(16) uint8_t rings[BW][LR * SSLOT];
    asm volatile("griddepcontrol.wait;" ::: "memory");
    asm volatile("griddepcontrol.launch_dependents;");
    const BandGeom &g = p.g;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int gx = (int)blockIdx.x % g.ngx, band = (int)blockIdx.x / g.ngx;
    const int s = gx * BW + warp;
    if (s >= g.nstrip) return;
    int y0, y1;
    band_rows(band, g.nband, p.rr.nrows, y0, y1);
    y0 += p.rr.oy0;
    y1 += p.rr.oy0;
    const bool cl = s < g.sx0, cr = s >= g.sx1, cy = band < g.by0 || band >= g.by1;
    const uint32_t ring = su32(rings[warp]);
    const int xs0 = s * SSTRIP, rows = y1 - y0;
    // Listing 3 per warp: Body warps run the unchecked body
    if (!cl && !cr && !cy) { sep_band_body<K, false, false, false>(p, ring, xs0, y0, rows, lane); return; }
    if (cy) {
        if (cl && cr) sep_band_body<K, true, true, true>(p, ring, xs0, y0, rows, lane);
        else if (cl) sep_band_body<K, true, false, true>(p, ring, xs0, y0, rows, lane);
        else if (cr) sep_band_body<K, false, true, true>(p, ring, xs0, y0, rows, lane);
        else sep_band_body<K, false, false, true>(p, ring, xs0, y0, rows, lane);
        return;
    }
    if (cl && cr) sep_band_body<K, true, true, false>(p, ring, xs0, y0, rows, lane);
    else if (cl) sep_band_body<K, true, false, false>(p, ring, xs0, y0, rows, lane);
    else sep_band_body<K, false, true, false>(p, ring, xs0, y0, rows, lane);
}

const void *sep_band_fn(int k)
{
    return k == 3 ? (const void *)k_sep_band<3> : k == 5 ? (const void *)k_sep_band<5> : (const void *)k_sep_band<7>;
}

int sep_band_blocks_per_sm(int k)
{
    static int nb[8] = {-1, -1, -1, -1, -1, -1, -1, -1};
    if (nb[k] < 0) {
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb[k], sep_band_fn(k), NTB, 0) != cudaSuccess) {
            cudaGetLastError();
            nb[k] = 0;
        }
    }
    return nb[k];
}

}  // namespace

int ispi_sep_band_blocks_per_sm(int k) { return sep_band_blocks_per_sm(k); }

// Eligibility: square separable 3 / 5 / 7 masks, 16-byte aligned rows in and out, w % 4 == 0,
// h >= 8 (one reflection at every edge), the whole image (no strips).
bool ispi_sep_band_ok(const float *img, int w, int h, int pitch, const float *out, int out_pitch, int mw, int mh)
{
    auto al = [](const void *q, long long pb) { return ((uintptr_t)q % 16) == 0 && (pb % 16) == 0; };
    return mw == mh && (mw == 3 || mw == 5 || mw == 7) && al(img, 4LL * pitch) && al(out, 4LL * out_pitch) &&
           w % 4 == 0 && w >= 8 && h >= 8;
}


void ispi_sep_band_shape(int w, int h, int k, int *tw, int *th)
{
    const BandGeom g = band_geom(w, h, w, w, ISP_CLAMP, k / 2, SSTRIP, sep_band_blocks_per_sm(k), bands_hint(), 185);
    *tw = SSTRIP;
    *th = (h + g.nband - 1) / g.nband;
}

cudaError_t ispi_sep_band(const float *img, int w, int h, int pitch, const float *row, const float *col, int k,
                          int mode, float cval, float *out, int out_pitch, cudaStream_t st, int bounds[4],
                          const RowRange *rr)
{
    SepBandParams p{};
    const int nrows = rr ? rr->nrows : h;
    p.g = band_geom(w, nrows, pitch, out_pitch, mode, k / 2, SSTRIP, sep_band_blocks_per_sm(k), bands_hint(), 185);
    p.g.h = h;
    p.rr = SepBandRows{0, h, 1, 1, 0, 0, h, nullptr, nullptr};
    if (rr) {
        p.rr = SepBandRows{rr->oy0, rr->nrows, rr->t_real, rr->b_real, rr->peer, rr->own_y0, rr->own_y1,
                           static_cast<const float *>(rr->peer_lo), static_cast<const float *>(rr->peer_hi)};
        // bands needing the T / B body: image edges are mapped, strip edges of the peer path
        // read the neighbours' buffers; a strip edge of the NCCL path reads its own halo rows
        const int hy = k / 2;
        auto top = [&](int b) {
            const int y0 = rr->oy0 + (int)((long long)b * nrows / p.g.nband);
            return (rr->t_real && y0 - hy < 0) || (rr->peer && y0 - hy < rr->own_y0);
        };
        auto bot = [&](int b) {
            const int y1 = rr->oy0 + (int)((long long)(b + 1) * nrows / p.g.nband);
            return (rr->b_real && y1 + hy > h) || (rr->peer && y1 + hy > rr->own_y1);
        };
        p.g.by0 = 0;
        while (p.g.by0 < p.g.nband && top(p.g.by0)) ++p.g.by0;
        p.g.by1 = p.g.by0;
        while (p.g.by1 < p.g.nband && !bot(p.g.by1)) ++p.g.by1;
    }
    p.img = img;
    p.out = out;
    p.cval = cval;
    std::memcpy(p.row, row, sizeof(float) * k);
    std::memcpy(p.col, col, sizeof(float) * k);
    bounds[0] = p.g.sx0; bounds[1] = std::max(p.g.sx0, p.g.sx1); bounds[2] = p.g.by0; bounds[3] = p.g.by1;
    return launch_band(sep_band_fn(k), &p, p.g.ngx * p.g.nband, st);
}
