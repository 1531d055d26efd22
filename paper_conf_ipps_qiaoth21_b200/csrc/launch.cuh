// launch.cuh -- template glue: pick the (op, mode, dispatch) kernel instance and launch it.
#pragma once
#include <mutex>
#include <unordered_map>

#include "isp_direct.cuh"
#include "isp_ops.cuh"
#include "isp_staged.cuh"
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
        default:
            if constexpr (MODE == MIRROR) return (const void *)k_direct<Op, MODE, DISP_NAIVE_GEN>;
            else return (const void *)k_direct<Op, MODE, DISP_NAIVE>;
        }
    } else {
        switch (disp) {
        case DISP_TMA:
            if constexpr (!Op::ROW_DIRECT) return (const void *)k_staged<Op>;  // one kernel, all modes
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
    return cudaLaunchKernel(fn, d.grid, d.block, args, d.smem, d.stream);
}

}  // namespace ispk
