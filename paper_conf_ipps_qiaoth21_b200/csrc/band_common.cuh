// band_common.cuh -- the warp-strip streaming skeleton shared by the band kernels
// (band_u8.cu: Laplace, Harris, fused cfg3; band_f32.cu: separable f32): the partition
// into warp strips x row bands with its Body rectangle (Listing 3 at warp granularity),
// row maps for T / B warps, the per-warp cp.async ring helpers and the launch.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <algorithm>
#include <cstdlib>

#include "../../include/isp.h"

namespace {

constexpr int BW = 4;                      // warps per CTA (adjacent strips of one band)
constexpr int NTB = 32 * BW;
constexpr int LR = 8;                      // ring slots per warp (power of 2): newest row + rows in flight


struct BandGeom {
    int w, h, pitch, out_pitch, mode;
    int nstrip, ngx, nband;  // strips, CTA columns, bands
    int sx0, sx1, by0, by1;  // Body strips [sx0, sx1), Body bands [by0, by1)
};

__device__ __forceinline__ uint32_t su32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void cpa_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cpa_wait()
{
    asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory");
}

__device__ __forceinline__ void band_rows(int b, int nb, int h, int &y0, int &y1)
{
    y0 = (int)((long long)b * h / nb);
    y1 = (int)((long long)(b + 1) * h / nb);
}

// Row y through the border pattern for an overshoot of at most the window's
// reach (one reflection: the launch requires h >= 8); -1: Constant, row outside.
template <bool CHK>
__device__ __forceinline__ int map_row1(int y, int h, int mode)
{
    if (!CHK || (y >= 0 && y < h)) return y;
    switch (mode) {
    case ISP_CLAMP: return y < 0 ? 0 : h - 1;
    case ISP_MIRROR: return y < 0 ? -y - 1 : 2 * h - 1 - y;
    case ISP_REPEAT: return y < 0 ? y + h : y - h;
    default: return -1;
    }
}

// 4-byte cp.async issued only by the lanes with `on` set (a predicated LDGSTS: the other
// lanes take no part, so the instruction costs one lane of shared-memory traffic)
__device__ __forceinline__ void cpa4p(uint32_t dst, const void *src, uint32_t on)
{
    asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %2, 0;\n\t@q cp.async.ca.shared.global [%0], [%1], 4;\n\t}" ::"r"(dst),
                 "l"(src), "r"(on)
                 : "memory");
}
__device__ __forceinline__ uint32_t lds32(uint32_t a)
{
    uint32_t v;
    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a) : "memory");
    return v;
}
__device__ __forceinline__ void sts32(uint32_t a, uint32_t v)
{
    asm volatile("st.shared.u32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}

int num_sms()
{
    static int n = 0;
    if (n == 0) {
        int dev = 0;
        if (cudaGetDevice(&dev) != cudaSuccess || cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev) !=
                                                      cudaSuccess) {
            cudaGetLastError();
            n = 148;
        }
    }
    return n;
}

// Strips, bands and the Body rectangle (hy rows of reach; a strip's right halo word lies
// past it, so a strip is Body iff it ends before the image's last column).
// waves100: how many waves of resident CTAs the bands fill, x 100 (the f32 band kernel
// measured best at ~1.85: DESIGN.md 7f; ISP_BAND_WAVES overrides it for experiments)
BandGeom band_geom(int w, int h, int pitch, int out_pitch, int mode, int hy, int strip, int per_sm, int bands_hint,
                   int waves100 = 100)
{
    BandGeom g{};
    g.w = w; g.h = h; g.pitch = pitch; g.out_pitch = out_pitch; g.mode = mode;
    g.nstrip = (w + strip - 1) / strip;
    g.ngx = (g.nstrip + BW - 1) / BW;
    int nb = bands_hint;
    if (nb <= 0) {
        if (const char *e = getenv("ISP_BAND_WAVES")) waves100 = std::max(10, atoi(e));
        nb = std::max(1, (int)((long long)waves100 * num_sms() * std::max(1, per_sm) / (100LL * g.ngx)));
    }
    g.nband = std::max(1, std::min(nb, h / (2 * hy + 2)));
    g.sx0 = 1;
    g.sx1 = (w - 1) / strip;
    g.by0 = g.nband;
    g.by1 = g.nband;
    for (int b = g.nband - 1; b >= 0; --b) {
        const int y0 = (int)((long long)b * h / g.nband), y1 = (int)((long long)(b + 1) * h / g.nband);
        if (y0 >= hy) g.by0 = b;
        if (y1 + hy > h) g.by1 = b;
    }
    if (g.by1 < g.by0) g.by1 = g.by0;
    return g;
}

cudaError_t launch_band(const void *fn, void *params, int nblocks, cudaStream_t st)
{
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3(nblocks);
    cfg.blockDim = dim3(NTB);
    cfg.stream = st;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    void *args[] = {params};
    return cudaLaunchKernelExC(&cfg, fn, args);
}

int bands_hint()
{
    const char *e = getenv("ISP_BAND_BANDS");
    return e ? atoi(e) : 0;
}

}  // namespace
