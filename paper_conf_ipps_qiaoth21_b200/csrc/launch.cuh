// launch.cuh -- template glue: pick the (op, mode, dispatch) kernel instance and launch it.
#pragma once
#include <cstdlib>
#include <mutex>
#include <unordered_map>

#include "isp_direct.cuh"
#include "isp_ops.cuh"
#include "isp_pstaged.cuh"
#include "kernels.h"

namespace ispk {

template <class Op, int MODE, bool DIRECT>
const void *kernel_for_disp(int disp)
{
    if constexpr (DIRECT) {
        switch (disp) {
        case DISP_BLOCK: return (const void *)k_direct<Op, MODE, DISP_BLOCK>;
        case DISP_WARP: return (const void *)k_direct<Op, MODE, DISP_BLOCK>;
        case DISP_NAIVE: return (const void *)k_direct<Op, MODE, DISP_NAIVE>;
        case DISP_TMA:
            if constexpr (Op::TILED) return (const void *)k_tile<Op, MODE>;
            else return nullptr;
        default:
            if constexpr (MODE == MIRROR) return (const void *)k_direct<Op, MODE, DISP_NAIVE_GEN>;
            else return (const void *)k_direct<Op, MODE, DISP_NAIVE>;
        }
    } else {
        switch (disp) {
        case DISP_TMA:
            if constexpr (!Op::ROW_DIRECT) return (const void *)k_pstaged<Op>;  // one kernel, all modes
            else return nullptr;
        case DISP_TMA_STATIC:
            if constexpr (!Op::ROW_DIRECT) return (const void *)k_staged<Op>;
            else return nullptr;
        case DISP_BLOCK: return (const void *)k_stencil<Op, MODE, DISP_BLOCK>;
        case DISP_WARP: return (const void *)k_stencil<Op, MODE, DISP_BLOCK>;
        case DISP_NAIVE: return (const void *)k_stencil<Op, MODE, DISP_NAIVE>;
        default:
            if constexpr (MODE == MIRROR) return (const void *)k_stencil<Op, MODE, DISP_NAIVE_GEN>;
            else return (const void *)k_stencil<Op, MODE, DISP_NAIVE>;
        }
    }
}

template <class Op, bool DIRECT = false>
const void *kernel_for(int mode, int disp)
{
    switch (mode) {
    case CLAMP: return kernel_for_disp<Op, CLAMP, DIRECT>(disp);
    case MIRROR: return kernel_for_disp<Op, MIRROR, DIRECT>(disp);
    case REPEAT: return kernel_for_disp<Op, REPEAT, DIRECT>(disp);
    case CONSTANT: return kernel_for_disp<Op, CONSTANT, DIRECT>(disp);
    }
    return nullptr;
}

inline bool pdl_enabled()
{
    static const bool on = [] {
        const char *e = getenv("ISP_PDL");
        return !(e && e[0] == '0');
    }();
    return on;
}

template <class P>
cudaError_t launch_params(const void *fn, const Desc &d, const P &p)
{
    if (!fn) return cudaErrorNotSupported;
    if (d.smem > 48 * 1024) {
        static std::mutex mu;
        static std::unordered_map<const void *, size_t> done;
        std::lock_guard<std::mutex> lk(mu);
        auto it = done.find(fn);
        if (it == done.end() || it->second < d.smem) {
            cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)d.smem);
            if (e != cudaSuccess) return e;
            done[fn] = d.smem;
        }
    }
    void *args[] = {const_cast<P *>(&p)};
    // programmatic dependent launch: the kernels call griddepcontrol.wait before touching
    // global memory, so their launch/prologue may overlap the previous kernel's tail
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = d.grid;
    cfg.blockDim = d.block;
    cfg.dynamicSmemBytes = d.smem;
    cfg.stream = d.stream;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = pdl_enabled() ? 1 : 0;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    return cudaLaunchKernelExC(&cfg, fn, args);
}

}  // namespace ispk
