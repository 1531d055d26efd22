// membench.cu -- B200 memory-path microbenchmarks used to choose the staged kernel's
// shape (not part of the library).  Build & run (on the GPU box):
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/membench tools/membench.cu
//   /tmp/membench
// Each line: pattern, parameters, GB/s (bytes moved / CUDA-event time, best of 5,
// rotating over buffers totalling > 2x L2).
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdio>
#include <vector>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { printf("CUDA %s @%d\n", cudaGetErrorString(e_), __LINE__); return 1; } } while (0)

__global__ void k_read_ldg(const float4 *__restrict__ a, size_t n4, float *sink)
{
    float acc = 0.f;
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n4; i += (size_t)gridDim.x * blockDim.x) {
        float4 v = __ldg(a + i);
        acc += v.x + v.y + v.z + v.w;
    }
    if (acc == 12345.f) *sink = acc;
}

__global__ void k_copy_ldg(const float4 *__restrict__ a, float4 *__restrict__ b, size_t n4)
{
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n4; i += (size_t)gridDim.x * blockDim.x)
        b[i] = __ldg(a + i);
}

__device__ __forceinline__ uint32_t su32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

// Each CTA streams `chunks` chunks of `chunk` bytes (chunk k of CTA c at address
// base + (c + k*gridDim.x) * stride) into a ring of S smem slots with cp.async.bulk.
// Optional: per chunk, 128 threads read the smem slot (mimics the consumer) and write
// it back to global (copy).
template <bool COPY>
__global__ void k_bulk(const char *__restrict__ src, char *__restrict__ dst, int chunk, size_t stride, int chunks,
                       int S)
{
    extern __shared__ __align__(128) unsigned char sm[];
    uint64_t *full = (uint64_t *)sm, *empty = full + 32;
    char *buf = (char *)(sm + 512);
    const int tid = threadIdx.x, nthr = blockDim.x - 32;
    if (tid == 0) {
        for (int s = 0; s < S; ++s) {
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&full[s])));
            asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su32(&empty[s])), "r"(nthr / 32));
        }
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    __syncthreads();
    if (tid >= nthr) {
        if (tid != nthr) return;
        for (int k = 0; k < chunks; ++k) {
            const int s = k % S;
            if (k >= S) {
                uint32_t par = ((k / S) - 1) & 1;
                asm volatile("{.reg .pred P; W: mbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1; @!P bra W;}" ::"r"(
                                 su32(&empty[s])), "r"(par) : "memory");
            }
            const char *g = src + (blockIdx.x + (size_t)k * gridDim.x) * stride;
            asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&full[s])), "r"(chunk) : "memory");
            asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                             su32(buf + (size_t)s * chunk)), "l"(g), "r"(chunk), "r"(su32(&full[s])) : "memory");
        }
        return;
    }
    for (int k = 0; k < chunks; ++k) {
        const int s = k % S;
        uint32_t par = (k / S) & 1;
        asm volatile("{.reg .pred P; W: mbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1; @!P bra W;}" ::"r"(
                         su32(&full[s])), "r"(par) : "memory");
        if (COPY) {
            char *d = dst + (blockIdx.x + (size_t)k * gridDim.x) * stride;
            for (int o = tid * 16; o < chunk; o += nthr * 16)
                *(float4 *)(d + o) = *(const float4 *)(buf + (size_t)s * chunk + o);
        }
        __syncwarp();
        if ((tid & 31) == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(su32(&empty[s])) : "memory");
    }
}

// Emulates the staged stencil's access pattern: CTA c reads column strip (c % ncol)
// of a 4096-row image with row pitch `pitch` bytes, rows [band*rpb, (band+1)*rpb),
// one `chunk`-byte bulk copy per row, S ring slots.
template <bool COPY>
__global__ void k_band(const char *__restrict__ src, char *__restrict__ dst, int chunk, size_t pitch, int ncol,
                       int rows, int S)
{
    extern __shared__ __align__(128) unsigned char sm[];
    uint64_t *full = (uint64_t *)sm, *empty = full + 32;
    char *buf = (char *)(sm + 512);
    const int tid = threadIdx.x, nthr = blockDim.x - 32;
    const int col = blockIdx.x % ncol, band = blockIdx.x / ncol, nband = gridDim.x / ncol;
    const int r0 = (int)((long long)band * rows / nband), r1 = (int)((long long)(band + 1) * rows / nband);
    const int chunks = r1 - r0;
    if (tid == 0) {
        for (int s = 0; s < S; ++s) {
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&full[s])));
            asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su32(&empty[s])), "r"(nthr / 32));
        }
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    __syncthreads();
    if (tid >= nthr) {
        if (tid != nthr) return;
        for (int k = 0; k < chunks; ++k) {
            const int s = k % S;
            if (k >= S) {
                uint32_t par = ((k / S) - 1) & 1;
                asm volatile("{.reg .pred P; W: mbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1; @!P bra W;}" ::"r"(
                                 su32(&empty[s])), "r"(par) : "memory");
            }
            const char *g = src + (size_t)(r0 + k) * pitch + (size_t)col * chunk;
            asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&full[s])), "r"(chunk) : "memory");
            asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                             su32(buf + (size_t)s * chunk)), "l"(g), "r"(chunk), "r"(su32(&full[s])) : "memory");
        }
        return;
    }
    for (int k = 0; k < chunks; ++k) {
        const int s = k % S;
        uint32_t par = (k / S) & 1;
        asm volatile("{.reg .pred P; W: mbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1; @!P bra W;}" ::"r"(
                         su32(&full[s])), "r"(par) : "memory");
        if (COPY) {
            char *d = dst + (size_t)(r0 + k) * pitch + (size_t)col * chunk;
            for (int o = tid * 16; o < chunk; o += nthr * 16)
                *(float4 *)(d + o) = *(const float4 *)(buf + (size_t)s * chunk + o);
        }
        __syncwarp();
        if ((tid & 31) == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(su32(&empty[s])) : "memory");
    }
}

int main()
{
    const size_t bytes = 64ull << 20;  // one 4096^2 f32 image
    const int NB = 8;                  // rotate over 8 in/out pairs = 1 GiB
    std::vector<char *> A(NB), B(NB);
    for (int i = 0; i < NB; ++i) {
        CK(cudaMalloc(&A[i], bytes));
        CK(cudaMalloc(&B[i], bytes));
        CK(cudaMemset(A[i], 1, bytes));
    }
    float *sink;
    CK(cudaMalloc(&sink, 4));
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    auto timeit = [&](auto fn, double moved) {
        float best = 1e30f;
        for (int rep = 0; rep < 5; ++rep) {
            fn(rep);  // warm
            cudaEventRecord(e0);
            for (int i = 0; i < NB; ++i) fn(i);
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            best = std::min(best, ms / NB);
        }
        return moved / (best * 1e-3) / 1e9;
    };
    const size_t n4 = bytes / 16;
    for (int bpsm : {4, 8, 16}) {
        int grid = sms * bpsm;
        double r = timeit([&](int i) { k_read_ldg<<<grid, 256>>>((const float4 *)A[i], n4, sink); }, bytes);
        double c = timeit([&](int i) { k_copy_ldg<<<grid, 256>>>((const float4 *)A[i], (float4 *)B[i], n4); }, 2.0 * bytes);
        printf("ldg       blocks/SM=%2d  read %7.1f GB/s   copy %7.1f GB/s\n", bpsm, r, c);
    }
    for (int chunk : {2048, 4096, 8192, 16384}) {
        for (int S : {4, 8, 16}) {
            for (int ctas : {2, 4, 7}) {
                const size_t smem = 512 + (size_t)S * chunk;
                if (smem > 220 * 1024 || (size_t)ctas * smem > 225 * 1024) continue;
                const int ncol = 16384 / chunk;
                const int grid = (sms * ctas / ncol) * ncol;
                CK(cudaFuncSetAttribute(k_band<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
                CK(cudaFuncSetAttribute(k_band<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
                double r = timeit([&](int i) { k_band<false><<<grid, 160, smem>>>(A[i], B[i], chunk, 16384, ncol, 4096, S); }, (double)bytes);
                double c = timeit([&](int i) { k_band<true><<<grid, 160, smem>>>(A[i], B[i], chunk, 16384, ncol, 4096, S); }, 2.0 * bytes);
                CK(cudaGetLastError());
                printf("band      chunk=%5d S=%2d ctas/SM=%d  read %7.1f GB/s   copy %7.1f GB/s\n", chunk, S, ctas, r, c);
            }
        }
    }
    for (int chunk : {2048, 4096, 8192, 16384}) {
        for (int S : {3, 8}) {
            for (int ctas : {2, 4, 7}) {
                const size_t smem = 512 + (size_t)S * chunk;
                if (smem > 220 * 1024 || (size_t)ctas * smem > 225 * 1024) continue;
                const int grid = sms * ctas;
                const size_t stride = chunk;  // contiguous chunks
                const int chunks = (int)(bytes / stride / grid);
                CK(cudaFuncSetAttribute(k_bulk<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
                CK(cudaFuncSetAttribute(k_bulk<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
                const double moved = (double)chunks * grid * chunk;
                double r = timeit([&](int i) { k_bulk<false><<<grid, 160, smem>>>(A[i], B[i], chunk, stride, chunks, S); }, moved);
                double c = timeit([&](int i) { k_bulk<true><<<grid, 160, smem>>>(A[i], B[i], chunk, stride, chunks, S); }, 2 * moved);
                CK(cudaGetLastError());
                printf("bulk      chunk=%5d S=%d ctas/SM=%d  read %7.1f GB/s   copy %7.1f GB/s\n", chunk, S, ctas, r, c);
            }
        }
    }
    return 0;
}
