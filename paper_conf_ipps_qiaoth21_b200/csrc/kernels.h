// kernels.h -- host-side interface between the C-ABI layer (api.cu) and the kernel
// instantiation units (k_*.cu).  Every family exposes:
//   const void *kfn_<family>(const Desc &)   kernel pointer (nullptr: not compiled)
//   cudaError_t run_<family>(const Desc &)   build params, launch on d.stream
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "isp_core.cuh"

namespace ispk {

struct U8RoundH {
    int divisor, shift, half;
};

struct Desc {
    Geom g;
    int mode, disp;
    dim3 grid, block;
    size_t smem;  // dynamic shared memory (TMA-staged family)
    cudaStream_t stream;
    const void *in0, *in1;
    void *out0, *out1, *out2;
    float cval_f;
    int cval_i;
    int mw, mh;
    int ax, ay;        // direct family: window anchor (cropped sparse masks, reading A31)
    int reach[4];      // non-zero footprint reach L, R, T, B (has_reach)
    int has_reach;
    const float *maskf, *rowf, *colf; // host
    const int *maski, *rowi, *coli;   // host
    U8RoundH rnd;
    long long thr;
    int tonemap;
    float kr;        // bilateral
    const float *ls; // bilateral log2 spatial weights (host)
    int dilation;
};

// streaming (compile-time window) families
const void *kfn_conv_f32(const Desc &);
cudaError_t run_conv_f32(const Desc &);
const void *kfn_sep_f32(const Desc &);
cudaError_t run_sep_f32(const Desc &);
const void *kfn_conv_u8(const Desc &);
cudaError_t run_conv_u8(const Desc &);
const void *kfn_sep_u8(const Desc &);
cudaError_t run_sep_u8(const Desc &);
const void *kfn_sobel(const Desc &);
cudaError_t run_sobel(const Desc &);
const void *kfn_laplace5(const Desc &);
cudaError_t run_laplace5(const Desc &);
const void *kfn_harris(const Desc &);
cudaError_t run_harris(const Desc &);
const void *kfn_atrous(const Desc &);
cudaError_t run_atrous(const Desc &);
// direct (runtime window) families
const void *kfn_dconv_f32(const Desc &);
cudaError_t run_dconv_f32(const Desc &);
const void *kfn_dconv_u8(const Desc &);
cudaError_t run_dconv_u8(const Desc &);
const void *kfn_bilateral(const Desc &);
cudaError_t run_bilateral(const Desc &);

// pixels per thread (x) of each family
constexpr int PX_F32 = 4, PX_U8 = kPxU8, PX_I16 = kPxI16, PX_DIRECT = 4;
#ifndef ISP_STAGED_WARPS
#define ISP_STAGED_WARPS 4
#endif
constexpr int STAGED_WARPS = ISP_STAGED_WARPS, STAGED_THREADS = 32 * (ISP_STAGED_WARPS + 1);
// shared-memory tiled kernel of the runtime-window ops (isp_direct.cuh k_tile)
constexpr int TILE_THREADS = 256, TILE_H = 16, TILE_PX = 4;

}  // namespace ispk
