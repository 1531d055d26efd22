// internal.h -- declarations shared by api.cu and shard.cu (not part of the C ABI).
#pragma once
#include "../../include/isp.h"

// Output row range of a launch: rows [oy0, oy0+nrows) of an image of height h whose
// resident input rows end at ylim; t_real / b_real: the range's top / bottom edge is a
// real image edge (else a strip edge whose neighbour rows arrive by halo exchange).
// peer (peer-direct halos): the strip's own rows are [own_y0, own_y1) of
// the buffer `img` points into; rows above / below come straight from the neighbour
// strips' memory (peer_lo / peer_hi, global-row addressed like img) -- the strip edges are
// then region edges too (their block rows select the neighbour buffer per row).
struct RowRange {
    int oy0, nrows, ylim, t_real, b_real;
    int peer = 0, own_y0 = 0, own_y1 = 0;
    const void *peer_lo = nullptr, *peer_hi = nullptr;
};

isp_status_t ispi_fail(isp_status_t s, const char *fmt, ...);
isp_status_t ispi_filter_f32(const float *img, int w, int h, int pitch, const float *mask, int mw, int mh,
                             int border_mode, float const_val, float *out, int out_pitch, isp_variant_t variant,
                             isp_stream_t stream, const RowRange *rr);
isp_status_t ispi_filter_u8(const uint8_t *img, int w, int h, int pitch, const int32_t *mask, int mw, int mh,
                            int32_t divisor, int border_mode, int const_val, uint8_t *out, int out_pitch,
                            isp_variant_t variant, isp_stream_t stream, const RowRange *rr);
isp_status_t ispi_filter_tex_f32(const float *img, int w, int h, int pitch, const float *mask, int mw, int mh,
                                 int border_mode, float const_val, float *out, int out_pitch, isp_stream_t stream);

// tile-staged u8 / i16 kernels (tile_u8.cu): the ISP_TMA variant of Laplace and Harris
#include <cuda_runtime.h>
bool ispi_tile_ok(const void *in0, const void *in1, int elem, int w, int h, int pitch, const void *out, int out_pitch);
void ispi_tile_shape(int *tw, int *th);
int ispi_tile_blocks_per_sm(int which);
cudaError_t ispi_laplace_tile(const uint8_t *img, int w, int h, int pitch, int mode, int cval, uint8_t *out,
                              int out_pitch, cudaStream_t st, int bounds[4]);
cudaError_t ispi_harris_tile(const int16_t *dx, const int16_t *dy, int w, int h, int pitch, int mode, int cval,
                             long long thr, uint8_t *out, int out_pitch, cudaStream_t st, int bounds[4]);

// warp-strip streaming band kernels (band_u8.cu): the ISP_TMA variant of Laplace and Harris
bool ispi_band_ok(const void *in, int w, int h, int pitch, const void *out, int out_pitch);
void ispi_band_shape(int w, int h, int *tw, int *th);
int ispi_band_blocks_per_sm(int which);   // 0: Laplace, 1: Harris, 2: Sobel
bool ispi_band_harris_ok(const void *dx, const void *dy, int w, int h, int pitch, const void *out, int out_pitch);
void ispi_band_harris_shape(int w, int h, int *tw, int *th);
cudaError_t ispi_harris_band(const int16_t *dx, const int16_t *dy, int w, int h, int pitch, int mode, int cval,
                             long long thr, uint8_t *out, int out_pitch, cudaStream_t st, int bounds[4]);
cudaError_t ispi_laplace_band(const uint8_t *img, int w, int h, int pitch, int mode, int cval, uint8_t *out,
                              int out_pitch, cudaStream_t st, int bounds[4]);
bool ispi_band_fused_ok(const void *img, int w, int h, int pitch, const void *mag, const void *lap, const void *har,
                        const void *dx, const void *dy, int out_pitch);
cudaError_t ispi_fused_band(const uint8_t *img, int w, int h, int pitch, int mode, int cval, int hcval, long long thr,
                            int16_t *dx, int16_t *dy, uint8_t *mag, uint8_t *lap, uint8_t *har, int out_pitch,
                            cudaStream_t st);
// separable f32 band kernel (band_f32.cu): ISP_TMA / AUTO of whole-image separable f32 masks
int ispi_sep_band_blocks_per_sm(int k);
bool ispi_sep_band_ok(const float *img, int w, int h, int pitch, const float *out, int out_pitch, int mw, int mh);
void ispi_sep_band_shape(int w, int h, int k, int *tw, int *th);
cudaError_t ispi_sep_band(const float *img, int w, int h, int pitch, const float *row, const float *col, int k,
                          int mode, float cval, float *out, int out_pitch, cudaStream_t st, int bounds[4],
                          const RowRange *rr = nullptr);
bool ispi_band_sobel_ok(const void *img, int w, int h, int pitch, const void *dx, const void *dy, const void *mag,
                        int out_pitch);
void ispi_band_sobel_shape(int w, int h, int *tw, int *th);
cudaError_t ispi_sobel_band(const uint8_t *img, int w, int h, int pitch, int mode, int cval, int16_t *dx, int16_t *dy,
                            uint8_t *mag, int out_pitch, cudaStream_t st, int bounds[4]);
bool ispi_sepu8_band_ok(const void *img, int w, int h, int pitch, const void *out, int out_pitch, int k,
                        const int *row, const int *col, int divisor);
void ispi_sepu8_band_shape(int w, int h, int k, int *tw, int *th);
int ispi_sepu8_band_blocks_per_sm(int k);
cudaError_t ispi_sepu8_band(const uint8_t *img, int w, int h, int pitch, int k, const int *row, const int *col,
                            int divisor, int mode, int cval, uint8_t *out, int out_pitch, cudaStream_t st, int bounds[4]);
