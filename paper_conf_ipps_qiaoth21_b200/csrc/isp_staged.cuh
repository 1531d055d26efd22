// isp_staged.cuh -- TMA-staged ISP kernels (bulk async copies + mbarrier pipeline).
//
// The B200-native form of the paper's fat kernel: one CTA per block of the
// partition (Listing 3 on blockIdx), four compute warps plus one producer
// warp.  The producer streams the CTA's input rows (tile + halo) into a ring of shared
// memory stages with cp.async.bulk (TMA engine, SASS UBLKCP) completing on mbarriers;
// the compute warps run the operator from shared memory with no bounds checks at all.
//
// Iteration space partitioning moves into the staging (reading A21): a Body CTA's rows
// and columns are all in bounds, so its producer issues plain bulk copies -- no index
// arithmetic per pixel; a border CTA maps only its out-of-bounds ROWS (T/B regions,
// once per row) and fixes up only its out-of-bounds COLUMNS (L/R regions, <= halo
// elements per row) through the border pattern.  The arithmetic the
// compute warps execute is identical to the streaming family (same op, same order),
// so results are bitwise identical to ISP_BLOCK / ISP_WARP / ISP_NAIVE.
#pragma once
#include "isp_ops.cuh"

namespace ispk {

#ifndef ISP_STAGED_WARPS
#define ISP_STAGED_WARPS 4
#endif
constexpr int kStagedComputeWarps = ISP_STAGED_WARPS;
constexpr int kStagedThreads = 32 * (kStagedComputeWarps + 1);
constexpr int kStagedMaxStages = 32;
constexpr int kStagedBarrierBytes = 512;  // full[32] + empty[32] mbarriers

__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_init(uint64_t *b, uint32_t count)
{
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t *b, uint32_t bytes)
{
    asm volatile("mbarrier.expect_tx.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t *b)
{
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(b)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *b, uint32_t parity)
{
    asm volatile(
        "{\n\t.reg .pred P1;\n\t"
        "LAB_WAIT:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t"
        "@P1 bra DONE;\n\t"
        "bra LAB_WAIT;\n\t"
        "DONE:\n\t}" ::"r"(smem_u32(b)),
        "r"(parity)
        : "memory");
}
__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, uint32_t bytes, uint64_t *bar)
{
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     smem_u32(dst)),
                 "l"(src), "r"(bytes), "r"(smem_u32(bar))
                 : "memory");
}
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
// 4-byte async copy global -> shared (LDGSTS) and an mbarrier arrive that fires when
// all of this thread's prior cp.async copies have landed (count not incremented).
__device__ __forceinline__ void cp_async4(void *dst, const void *src)
{
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async_mbar_arrive_noinc(uint64_t *b)
{
    asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];" ::"r"(smem_u32(b)) : "memory");
}

// Global column the fix-up of column x reads (x outside the bulk-copied range), or -1
// when no stored output reads it (beyond the window's reach: left as is).
template <class Op, int MODE, int CK>
__device__ __forceinline__ int fixup_source(int x, const Geom &g)
{
    if (x >= 0 && x < g.w) return x;
    if (x < -Op::HX || x >= g.w + Op::HX) return -1;
    if constexpr ((CK & CK_L) != 0) {
        if (x < 0) return bmap<MODE, true, false, false>(x, g.w);
    }
    if constexpr ((CK & CK_R) != 0) {
        if (x >= g.w) return bmap<MODE, false, true, false>(x, g.w);
    }
    return -1;
}
__device__ __forceinline__ void fence_mbar_init() { asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory"); }

template <int N>
__device__ __forceinline__ void lds_words(uint32_t *dst, const void *src)
{
    if constexpr (N == 4) {
        const uint4 q = *reinterpret_cast<const uint4 *>(src);
        dst[0] = q.x; dst[1] = q.y; dst[2] = q.z; dst[3] = q.w;
    } else if constexpr (N == 2) {
        const uint2 q = *reinterpret_cast<const uint2 *>(src);
        dst[0] = q.x; dst[1] = q.y;
    } else {
        dst[0] = *reinterpret_cast<const uint32_t *>(src);
    }
}

// One row segment from shared memory: srow points at this thread's column x0.
template <class Op>
__device__ __forceinline__ void load_row_smem(const typename Op::Tin *const (&srow)[Op::NIN], RawRow<Op> &rr)
{
    using T = typename Op::Tin;
    using U = VecUse<Op>;
    constexpr int PX = Op::PX, NV = RawRow<Op>::NV, WPV = U::WPV;
#pragma unroll
    for (int c = 0; c < Op::NIN; ++c)
#pragma unroll
        for (int v = -NV; v <= NV; ++v) {
            if (U::lo(v) >= PX) continue;
            uint32_t(&wv)[WPV] = rr.w[c][v + NV];
            const int fw = U::first_word(v), n = U::nwords(v);
            const char *src = reinterpret_cast<const char *>(srow[c] + v * PX) + 4 * fw;
            if constexpr (WPV >= 4) {
                if (n == 4) { lds_words<4>(&wv[fw], src); continue; }
            }
            if constexpr (WPV >= 2) {
                if (n == 2) { lds_words<2>(&wv[fw], src); continue; }
            }
            lds_words<1>(&wv[fw], src);
        }
}

// Value of global column x of a row that needs a fix-up (x outside the bulk-copied
// range): in-bounds tail, border pattern, or don't-care beyond the window's reach.
template <class Op, int MODE, int CK>
__device__ __forceinline__ typename Op::Tin fixup_value(const typename Op::Tin *__restrict__ src, int x,
                                                        const Geom &g, typename Op::Tin cval)
{
    using T = typename Op::Tin;
    if (x >= 0 && x < g.w) return __ldg(src + x);
    if (x < -Op::HX || x >= g.w + Op::HX) return T(0);  // no stored output reads it
    if constexpr (MODE == CONSTANT) {
        return cval;
    } else {
        if constexpr ((CK & CK_L) != 0) {
            if (x < 0) return __ldg(src + bmap<MODE, true, false, false>(x, g.w));
        }
        if constexpr ((CK & CK_R) != 0) {
            if (x >= g.w) return __ldg(src + bmap<MODE, false, true, false>(x, g.w));
        }
        return T(0);
    }
}

// Clamp and Mirror columns beyond a side are copies of columns inside the tile (and
// Constant columns are C), so
// when the width is a whole number of vectors (no partial vector at the right edge) the
// compute warps rebuild them in registers (staged_edge_fix) and the producer issues no
// column fix-ups at all: L/R CTAs then stage exactly like Body CTAs.
__device__ __forceinline__ bool consumer_fix(const Geom &g, int px)
{
    return g.mode != REPEAT && g.w % px == 0 && g.w_al == g.w && g.dbg != 5;
}

template <class Op, int CK>
__device__ __forceinline__ void staged_edge_fix(const Geom &g, int x0, typename Op::Tin (&seg)[Op::NIN][Op::PX + 2 * Op::HX],
                                                typename Op::Tin cval)
{
    constexpr int PX = Op::PX, HX = Op::HX;
    const bool mirror = g.mode == MIRROR, cst = g.mode == CONSTANT;
#pragma unroll
    for (int c = 0; c < Op::NIN; ++c) {
        if constexpr ((CK & CK_L) != 0) {
            if (x0 == 0) {  // columns -HX..-1 <- 0 (Clamp) / HX-1..0 (Mirror)
#pragma unroll
                for (int k = 0; k < HX; ++k) seg[c][k] = cst ? cval : mirror ? seg[c][2 * HX - 1 - k] : seg[c][HX];
            }
        }
        if constexpr ((CK & CK_R) != 0) {
            if (x0 + PX == g.w) {  // columns w..w+HX-1 <- w-1 (Clamp) / w-1..w-HX (Mirror)
#pragma unroll
                for (int t = 0; t < HX; ++t)
                    seg[c][HX + PX + t] = cst ? cval : mirror ? seg[c][HX + PX - 1 - t] : seg[c][HX + PX - 1];
            }
        }
    }
}

// Producer warp of a staged CTA (the only mode-dependent code: row maps, fix-ups).
template <class Op, int MODE, int CK>
__device__ __forceinline__ void staged_producer(const typename Op::Params &p, uint64_t *full, uint64_t *empty,
                                                typename Op::Tin *buf, int y0, int nr, int X0)
{
    using T = typename Op::Tin;
    constexpr int HY = Op::HY, PX = Op::PX, NIN = Op::NIN;
    constexpr int TW = kStagedComputeWarps * 32 * PX;
    constexpr bool ASYNC_FIX = (CK & (CK_L | CK_R)) != 0 && sizeof(T) == 4 && MODE != CONSTANT;
    const Geom &g = p.g;
    const int S = g.stages, SW = g.sw, HXA = g.hxa, RS = g.rs;
    const int lane = threadIdx.x & 31;
    const int XS = X0 - HXA;
    const size_t row_elems = (size_t)NIN * SW, slot_elems = (size_t)RS * row_elems;
    // ---------------- producer warp: RS input rows per ring slot ----------------
    int s = 0, nfill = 0;
    uint32_t ph = 0;
    for (int f0 = 0; f0 < nr; f0 += RS, ++nfill) {
        if (nfill >= S) mbar_wait(&empty[s], ph ^ 1);
        const int nrow = min(RS, nr - f0);
        T *sb = buf + (size_t)s * slot_elems;
        uint32_t bytes = 0;
        for (int k = 0; k < nrow; ++k) {
            bool rowok;
            map_row<MODE, CK>(y0 - HY + f0 + k, g, rowok);
            int cs = XS, ce = X0 + TW + HXA;
            if constexpr ((CK & CK_L) != 0) cs = max(cs, 0);
            if constexpr ((CK & CK_R) != 0) ce = min(ce, g.w_al);
            if (!(MODE == CONSTANT && !rowok) && ce > cs) bytes += (uint32_t)(ce - cs) * (uint32_t)sizeof(T) * NIN;
        }
        if (lane == 0) mbar_expect_tx(&full[s], bytes);
        for (int k = 0; k < nrow; ++k) {
            bool rowok;
            const int yy = map_row<MODE, CK>(y0 - HY + f0 + k, g, rowok);
            int cs = XS, ce = X0 + TW + HXA;
            if constexpr ((CK & CK_L) != 0) cs = max(cs, 0);
            if constexpr ((CK & CK_R) != 0) ce = min(ce, g.w_al);
            if (MODE == CONSTANT && !rowok) ce = cs;  // whole row = C
            T *rb = sb + (size_t)k * row_elems;
            if (lane == 0 && ce > cs)
#pragma unroll
                for (int c = 0; c < NIN; ++c)
                    bulk_g2s(rb + (size_t)c * SW + (cs - XS), row_base<CK>(p.in[c], yy, g) + cs,
                             (uint32_t)(ce - cs) * (uint32_t)sizeof(T), &full[s]);
            if (CK != 0 && g.dbg != 4) {
                // column fix-ups unless the compute warps rebuild the edge columns
                const bool colfix = !((CK & (CK_L | CK_R)) && consumer_fix(g, PX));
                // border fix-ups, this region's sides only (<= HXA columns per row):
                // cp.async of the pattern's source column (4-byte types), else a
                // synchronous copy; Constant: the constant
#pragma unroll
                for (int c = 0; c < NIN; ++c) {
                    T *dst = rb + (size_t)c * SW;
                    if (MODE == CONSTANT && !rowok) {
                        for (int x = lane; x < SW; x += 32) dst[x] = p.cval;
                        continue;
                    }
                    if (!colfix) continue;
                    const T *src = row_base<CK>(p.in[c], yy, g);
                    auto fix = [&](int x) {
                        if constexpr (MODE == CONSTANT) {
                            dst[x - XS] = (x >= 0 && x < g.w) ? __ldg(src + x) : p.cval;
                        } else {
                            const int xs = fixup_source<Op, MODE, CK>(x, g);
                            if (xs < 0) return;
                            if constexpr (ASYNC_FIX) cp_async4(dst + (x - XS), src + xs);
                            else dst[x - XS] = __ldg(src + xs);
                        }
                    };
                    if constexpr ((CK & CK_L) != 0)
                        for (int x = XS + lane; x < cs; x += 32) fix(x);
                    if constexpr ((CK & CK_R) != 0)
                        for (int x = ce + lane; x < X0 + TW + HXA; x += 32) fix(x);
                }
            }
        }
        if constexpr (ASYNC_FIX) {
            if (g.dbg != 4 && !consumer_fix(g, PX)) cp_async_mbar_arrive_noinc(&full[s]);
        }
        if constexpr (MODE == CONSTANT && (CK & (CK_T | CK_B)) != 0)
            fence_proxy_async();  // generic row fills before later bulk (async-proxy) writes
        __syncwarp();
        if (lane == 0) mbar_arrive(&full[s]);
        if (++s == S) { s = 0; ph ^= 1; }
    }
}

template <class Op, int CK>
__device__ __forceinline__ void staged_body(const typename Op::Params &p, unsigned char *smem)
{
    using T = typename Op::Tin;
    constexpr int MH = Op::MH, HY = Op::HY, PX = Op::PX, NIN = Op::NIN, SEGW = PX + 2 * Op::HX;
    constexpr int NWC = kStagedComputeWarps, TW = NWC * 32 * PX;
    const Geom &g = p.g;
    const int S = g.stages, SW = g.sw, HXA = g.hxa;
    uint64_t *full = reinterpret_cast<uint64_t *>(smem);
    uint64_t *empty = full + kStagedMaxStages;
    T *buf = reinterpret_cast<T *>(smem + kStagedBarrierBytes);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    int y0, rows;
    block_rows(g, blockIdx.y, gridDim.y, y0, rows);
    const int nr = rows + 2 * HY;            // input rows of this CTA (one ring slot each)
    const int X0 = blockIdx.x * TW;          // first output column of the CTA
    const int RS = g.rs;                     // rows per ring slot
    const size_t row_elems = (size_t)NIN * SW, slot_elems = (size_t)RS * row_elems;

    // L/R CTAs of 4-byte types fetch their fix-up columns with cp.async: every producer
    // lane then arrives on the full barrier when its copies land (32 extra arrivals)
    const bool async_fix = (CK & (CK_L | CK_R)) != 0 && sizeof(T) == 4 && g.mode != CONSTANT;
    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) {
            mbar_init(&full[s], async_fix && g.dbg != 4 && !consumer_fix(g, Op::PX) ? 33 : 1);
            mbar_init(&empty[s], NWC);
        }
        fence_mbar_init();
    }
    __syncthreads();
    pdl_wait();  // the prologue above overlaps the previous kernel's tail (PDL)
    if (g.trace && threadIdx.x == 0) g.trace[4ull * (blockIdx.y * gridDim.x + blockIdx.x) + 3] = gtimer();

    if (warp == NWC) {
        switch (g.mode) {  // the border pattern is a runtime parameter of the staged kernel
        case CLAMP: staged_producer<Op, CLAMP, CK>(p, full, empty, buf, y0, nr, X0); break;
        case MIRROR: staged_producer<Op, MIRROR, CK>(p, full, empty, buf, y0, nr, X0); break;
        case REPEAT: staged_producer<Op, REPEAT, CK>(p, full, empty, buf, y0, nr, X0); break;
        default: staged_producer<Op, CONSTANT, CK>(p, full, empty, buf, y0, nr, X0); break;
        }
        return;
    }

    // ---------------- compute warps ----------------
    const int xoff = (warp * 32 + lane) * PX;  // column within the tile
    const int x0 = X0 + xoff;
    typename Op::A acc[MH];
#pragma unroll
    for (int k = 0; k < MH; ++k) Op::zero(acc[k]);
    int s = 0, kr = 0;
    uint32_t ph = 0;
    for (int r0 = 0; r0 < nr; r0 += MH) {
#pragma unroll
        for (int k = 0; k < MH; ++k) {
            const int r = r0 + k;
            if (r < nr) {
                if (kr == 0) mbar_wait(&full[s], ph);
                const T *rb = buf + (size_t)s * slot_elems + (size_t)kr * row_elems;
                RawRow<Op> rr;
                if (g.dbg != 1) {
                    const T *srow[NIN];
#pragma unroll
                    for (int c = 0; c < NIN; ++c) srow[c] = rb + (size_t)c * SW + HXA + xoff;
                    load_row_smem<Op>(srow, rr);
                }
                if (++kr == RS || r == nr - 1) {
                    __syncwarp();
                    if (lane == 0) mbar_arrive(&empty[s]);  // release: the slot's rows are in registers
                    kr = 0;
                    if (++s == S) { s = 0; ph ^= 1; }
                }
                if (g.dbg == 1) continue;
                T seg[NIN][SEGW];
                unpack_row<Op>(rr, seg);
                if constexpr ((CK & (CK_L | CK_R)) != 0) {
                    if (consumer_fix(g, PX)) staged_edge_fix<Op, CK>(g, x0, seg, p.cval);
                }
                typename Op::H hs;
                Op::hrow(p, seg, hs);
                // every tap unconditionally: j == 0 initialises the row's accumulator, so
                // rows before the strip (o < 0) or past it (o >= rows) only touch slots
                // that are re-initialised before use or never stored
                Op::template vacc<true>(p, 0, hs, acc[k]);
#pragma unroll
                for (int j = 1; j < MH; ++j) {
                    if (!Op::row_used(j)) continue;
                    Op::template vacc<false>(p, j, hs, acc[(k - j + MH) % MH]);
                }
                const int o = r - (MH - 1);
                if (o >= 0 && g.dbg != 2) Op::template store<CK & CK_R>(p, acc[(k + 1) % MH], x0, y0 + o);
            }
        }
    }
}

// The TMA-staged fat kernel: Listing 3 on (blockIdx.x, blockIdx.y) with the staging
// bounds of Geom (BH_L/BH_R from the aligned halo HXA, reading A21).
template <class Op>
__global__ void __launch_bounds__(kStagedThreads) k_staged(const __grid_constant__ typename Op::Params p)
{
    extern __shared__ __align__(128) unsigned char smem[];
    pdl_launch_dependents();
    // dbg 8 (timing experiment only, wrong borders): every CTA runs the Body path
    const int rg = p.g.dbg == 8 ? RG_BODY : region_of(p.g, blockIdx.x, blockIdx.y, 0, false);
    const unsigned long long t0 = p.g.trace ? gtimer() : 0;
    switch (rg) {
    case RG_TL: staged_body<Op, region_checks(RG_TL)>(p, smem); break;
    case RG_TR: staged_body<Op, region_checks(RG_TR)>(p, smem); break;
    case RG_T: staged_body<Op, region_checks(RG_T)>(p, smem); break;
    case RG_BL: staged_body<Op, region_checks(RG_BL)>(p, smem); break;
    case RG_BR: staged_body<Op, region_checks(RG_BR)>(p, smem); break;
    case RG_B: staged_body<Op, region_checks(RG_B)>(p, smem); break;
    case RG_R: staged_body<Op, region_checks(RG_R)>(p, smem); break;
    case RG_L: staged_body<Op, region_checks(RG_L)>(p, smem); break;
    default: staged_body<Op, 0>(p, smem); break;
    }
    if (p.g.trace && threadIdx.x == 0) {  // compute warp 0 finished its rows
        unsigned long long *t = p.g.trace + 4ull * (blockIdx.y * gridDim.x + blockIdx.x);
        t[0] = (unsigned long long)smid() | ((unsigned long long)rg << 16) | ((unsigned long long)blockIdx.y << 32) |
               ((unsigned long long)blockIdx.x << 48);
        t[1] = t0;
        t[2] = gtimer();
    }
}

}  // namespace ispk
