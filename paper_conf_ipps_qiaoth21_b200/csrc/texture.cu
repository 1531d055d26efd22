// texture.cu -- ablation: border handling by the TEXTURE
// hardware instead of iteration space partitioning.  The paper cites texture memory as
// the hardware alternative ("textures ... are bound to the image size and not supported
// for sub-regions"); this variant reads every tap through a texture object over the
// caller's pitch-linear image whose address mode IS the border pattern:
//
//   Clamp    -> cudaAddressModeClamp  (unnormalised coordinates)
//   Constant -> cudaAddressModeBorder with borderColor = C
//   Repeat   -> cudaAddressModeWrap   (normalised coordinates; periodic for any offset)
//   Mirror   -> cudaAddressModeMirror (normalised; symmetric with the edge duplicated,
//               i.e. reading A4's -1 -> 0, period 2N)
//
// Point sampling at texel centres, one output pixel per thread, taps in row-major order
// with one FMA chain from 0 -- the direct family's arithmetic (DOpConvF32), so the
// results are those of isp_filter_ex's 2-D form.  Not a product path: ISP_TEX exists to
// time the alternative the paper argues against.
#include <cuda_runtime.h>

#include <cstring>
#include <map>
#include <mutex>
#include <tuple>

#include "../../include/isp.h"
#include "internal.h"

namespace {

constexpr int kTexMaxTaps = 31 * 31;

struct TexParams {
    cudaTextureObject_t tex;
    int w, h, mw, mh, ax, ay, out_pitch, normalized;
    float inv_w, inv_h;
    float *out;
    float mask[kTexMaxTaps];
};

__global__ void __launch_bounds__(256) k_tex(const __grid_constant__ TexParams p)
{
    const int x = blockIdx.x * 32 + threadIdx.x, y = blockIdx.y * 8 + threadIdx.y;
    if (x >= p.w || y >= p.h) return;
    float acc = 0.f;
    for (int j = 0; j < p.mh; ++j) {
        const float yc = (float)(y + j - p.ay) + 0.5f;
        for (int i = 0; i < p.mw; ++i) {
            const float xc = (float)(x + i - p.ax) + 0.5f;
            const float v = p.normalized ? tex2D<float>(p.tex, xc * p.inv_w, yc * p.inv_h) : tex2D<float>(p.tex, xc, yc);
            acc = fmaf(p.mask[j * p.mw + i], v, acc);
        }
    }
    p.out[(size_t)y * p.out_pitch + x] = acc;
}

// Texture objects are cached per (image, geometry, pattern, constant): a launch captured in
// a CUDA graph keeps its object valid for every replay.
std::mutex g_mu;
std::map<std::tuple<const void *, int, int, int, int, uint32_t, int>, cudaTextureObject_t> g_cache;

isp_status_t tex_object(const float *img, int w, int h, int pitch, int mode, float cval, cudaTextureObject_t *out)
{
    int dev = 0;
    cudaGetDevice(&dev);
    uint32_t cbits;
    std::memcpy(&cbits, &cval, 4);
    const auto key = std::make_tuple((const void *)img, w, h, pitch, mode, mode == ISP_CONSTANT ? cbits : 0u, dev);
    std::lock_guard<std::mutex> lk(g_mu);
    auto it = g_cache.find(key);
    if (it != g_cache.end()) {
        *out = it->second;
        return ISP_OK;
    }
    int talign = 0, palign = 0;
    cudaDeviceGetAttribute(&talign, cudaDevAttrTextureAlignment, dev);
    cudaDeviceGetAttribute(&palign, cudaDevAttrTexturePitchAlignment, dev);
    if ((talign > 0 && (uintptr_t)img % talign) || (palign > 0 && ((size_t)pitch * 4) % palign))
        return ispi_fail(ISP_EUNSUPPORTED, "ISP_TEX: image base / pitch not texture-aligned (%d / %d B)", talign, palign);
    cudaResourceDesc rd{};
    rd.resType = cudaResourceTypePitch2D;
    rd.res.pitch2D.devPtr = const_cast<float *>(img);
    rd.res.pitch2D.desc = cudaCreateChannelDesc<float>();
    rd.res.pitch2D.width = w;
    rd.res.pitch2D.height = h;
    rd.res.pitch2D.pitchInBytes = (size_t)pitch * 4;
    cudaTextureDesc td{};
    const cudaTextureAddressMode am = mode == ISP_CLAMP ? cudaAddressModeClamp
                                      : mode == ISP_MIRROR ? cudaAddressModeMirror
                                      : mode == ISP_REPEAT ? cudaAddressModeWrap : cudaAddressModeBorder;
    td.addressMode[0] = td.addressMode[1] = am;
    td.filterMode = cudaFilterModePoint;
    td.readMode = cudaReadModeElementType;
    td.normalizedCoords = (mode == ISP_MIRROR || mode == ISP_REPEAT) ? 1 : 0;
    td.borderColor[0] = td.borderColor[1] = td.borderColor[2] = td.borderColor[3] = cval;
    cudaTextureObject_t t = 0;
    cudaError_t e = cudaCreateTextureObject(&t, &rd, &td, nullptr);
    if (e != cudaSuccess) return ispi_fail(ISP_ECUDA, "cudaCreateTextureObject: %s", cudaGetErrorString(e));
    if (g_cache.size() > 256) {   // bound the cache (objects of old buffers)
        for (auto &kv : g_cache) cudaDestroyTextureObject(kv.second);
        g_cache.clear();
    }
    g_cache[key] = t;
    *out = t;
    return ISP_OK;
}

}  // namespace

isp_status_t ispi_filter_tex_f32(const float *img, int w, int h, int pitch, const float *mask, int mw, int mh,
                                 int border_mode, float const_val, float *out, int out_pitch, isp_stream_t stream)
{
    TexParams p{};
    isp_status_t s = tex_object(img, w, h, pitch, border_mode, const_val, &p.tex);
    if (s != ISP_OK) return s;
    p.w = w;
    p.h = h;
    p.mw = mw;
    p.mh = mh;
    p.ax = mw / 2;
    p.ay = mh / 2;
    p.out_pitch = out_pitch;
    p.normalized = (border_mode == ISP_MIRROR || border_mode == ISP_REPEAT) ? 1 : 0;
    p.inv_w = 1.0f / (float)w;
    p.inv_h = 1.0f / (float)h;
    p.out = out;
    std::memcpy(p.mask, mask, sizeof(float) * mw * mh);
    const dim3 grid((w + 31) / 32, (h + 7) / 8), block(32, 8);
    k_tex<<<grid, block, 0, (cudaStream_t)stream>>>(p);
    const cudaError_t e = cudaGetLastError();
    return e == cudaSuccess ? ISP_OK : ispi_fail(ISP_ECUDA, "k_tex: %s", cudaGetErrorString(e));
}
