// isp_pstaged.cuh -- persistent TMA-staged ISP kernels with a dynamic row-chunk scheduler.
//
// Same operator code, region logic and staging rules as isp_staged.cuh (reading A21:
// ISP lives in the staging -- Body units bulk-copy their rows unchecked, T/B units map
// rows, L/R units fix up columns), but the partition is the paper's uniform one (Eq. 2
// with tiles of TW x CH pixels, Listing 3 on the tile grid) and the tiles ("units") are
// handed out at run time:
//
//   * one or two resident CTAs per SM (grid <= #SMs x CTAs/SM), each = NWC compute
//     warps + 1 producer warp; the producer claims units with an atomic counter in
//     row-major order (tile column fastest), so the whole GPU sweeps the image top to
//     bottom as one front;
//   * a unit's halo rows (HY above and below) are the neighbouring units' rows, which
//     the front read moments before: they come from L2, not DRAM (the static one-wave
//     split of isp_staged.cuh re-read ~12 % of the image from DRAM on cfg2);
//   * load balance is per unit (~1 us), not per CTA, so no CTA tail;
//   * the ring of single-row shared-memory slots runs continuously across units: every
//     slot carries its unit id, the consumers switch region bodies per unit.
//
// Each unit's region is Listing 3 on (unit column, unit row) with Eq. (2) bounds for the
// TW x CH tile (reading A2/A21), so the dispatch is warp-uniform and the Body unit's
// code has no checks.  Results are bitwise identical to every other variant (same op,
// same arithmetic order).
#pragma once
#include "isp_staged.cuh"

namespace ispk {


struct PUnit {
    int x0, y0, rows, rg;
};

__device__ __forceinline__ PUnit punit_of(const Geom &g, int u)
{
    const int bx = u % g.nux, by = u / g.nux;
    PUnit r;
    r.x0 = bx * g.nwc * 32 * g.px;
    r.y0 = g.oy0 + by * g.ty;
    r.rows = min(g.ty, g.y_end - r.y0);
    r.rg = g.dbg == 8 ? RG_BODY : region_of(g, bx, by, 0, false);  // dbg 8: timing experiment
    return r;
}

// Producer: all input rows of one unit into consecutive ring slots.
template <class Op, int MODE, int CK>
__device__ __forceinline__ void pstaged_produce(const typename Op::Params &p, uint64_t *full, uint64_t *empty,
                                                int4 *meta, typename Op::Tin *buf, int &s, uint32_t &ph,
                                                long long &nfill, int u, const PUnit &un)
{
    using T = typename Op::Tin;
    constexpr int HY = Op::HY, PX = Op::PX, NIN = Op::NIN;
    constexpr bool FIX4 = sizeof(T) == 4 && MODE != CONSTANT;
    const Geom &g = p.g;
    const int S = g.stages, SW = g.sw, HXA = g.hxa;
    const int TW = g.nwc * 32 * PX;
    const int lane = threadIdx.x & 31;
    const int X0 = un.x0, XS = X0 - HXA;
    const int nr = un.rows + 2 * HY;
    const size_t row_elems = (size_t)NIN * SW;
    const bool colfix = (CK & (CK_L | CK_R)) != 0 && !consumer_fix(g, PX);
    // Repeat with a whole number of 16-B vectors per row: the wrapped halo columns are
    // contiguous, so they arrive as a second bulk copy instead of element fix-ups
    const bool rep_bulk = MODE == REPEAT && g.w == g.w_al && g.hxa <= g.w;
    for (int k = 0; k < nr; ++k) {
        if (nfill >= S) mbar_wait(&empty[s], ph ^ 1);
        ++nfill;
        bool rowok;
        const int yy = map_row<MODE, CK>(un.y0 - HY + k, g, rowok);
        int cs = XS, ce = X0 + TW + HXA;
        if constexpr ((CK & CK_L) != 0) cs = max(cs, 0);
        if constexpr ((CK & CK_R) != 0) ce = min(ce, g.w_al);
        if (MODE == CONSTANT && !rowok) ce = cs;
        // wrapped Repeat halo segments (bulk): left [XS, 0) <- [w + XS, w); right [w, end) <- [0, end - w)
        int wl = 0, wr = 0;
        if constexpr (MODE == REPEAT && (CK & (CK_L | CK_R)) != 0) {
            if (rep_bulk) {
                // columns beyond w + HXA feed no stored output: not fetched (wr <= HXA <= w)
                if ((CK & CK_L) != 0 && XS < 0) wl = -XS;
                if ((CK & CK_R) != 0 && X0 + TW + HXA > g.w) wr = min(X0 + TW + HXA, g.w + HXA) - g.w;
            }
        }
        T *rb = buf + (size_t)s * row_elems;
        if (lane == 0) {
            meta[s] = make_int4(u, k, nr, 0);
            const uint32_t bytes = (uint32_t)(max(ce - cs, 0) + wl + wr) * (uint32_t)sizeof(T) * NIN;
            mbar_expect_tx(&full[s], bytes);
            const T *const *in = p.in;
#pragma unroll
            for (int c = 0; c < NIN; ++c) {
                const T *src = row_base<CK>(in[c], yy, g);
                T *dst = rb + (size_t)c * SW;
                if (ce > cs) bulk_g2s(dst + (cs - XS), src + cs, (uint32_t)(ce - cs) * (uint32_t)sizeof(T), &full[s]);
                if (wl) bulk_g2s(dst, src + g.w - wl, (uint32_t)wl * (uint32_t)sizeof(T), &full[s]);
                if (wr) bulk_g2s(dst + (g.w - XS), src, (uint32_t)wr * (uint32_t)sizeof(T), &full[s]);
            }
        }
        if (CK != 0) {
#pragma unroll
            for (int c = 0; c < NIN; ++c) {
                T *dst = rb + (size_t)c * SW;
                if (MODE == CONSTANT && !rowok) {
                    for (int x = lane; x < SW; x += 32) dst[x] = p.cval;
                    continue;
                }
                if (!colfix || rep_bulk) continue;
                const T *src = row_base<CK>(p.in[c], yy, g);
                auto fix = [&](int x) {
                    if constexpr (MODE == CONSTANT) {
                        dst[x - XS] = (x >= 0 && x < g.w) ? __ldg(src + x) : p.cval;
                    } else {
                        const int xs = fixup_source<Op, MODE, CK>(x, g);
                        if (xs < 0) return;
                        if constexpr (FIX4) cp_async4(dst + (x - XS), src + xs);
                        else dst[x - XS] = __ldg(src + xs);
                    }
                };
                if constexpr ((CK & CK_L) != 0)
                    for (int x = XS + lane; x < cs; x += 32) fix(x);
                if constexpr ((CK & CK_R) != 0)
                    for (int x = ce + lane; x < X0 + TW + HXA; x += 32) fix(x);
            }
        }
        if constexpr (MODE == CONSTANT && (CK & (CK_T | CK_B)) != 0)
            fence_proxy_async();  // generic row fills before later bulk (async-proxy) writes of this slot
        // every producer lane arrives when its own cp.async fix-ups (if any) have landed;
        // lane 0's arrive also carries the expect_tx of the bulk copies
        cp_async_mbar_arrive_noinc(&full[s]);
        if (lane == 0) mbar_arrive(&full[s]);
        if (++s == S) { s = 0; ph ^= 1; }
    }
}

// Consumer warps: all rows of one unit (the first slot's meta has been read).
template <class Op, int CK>
__device__ __forceinline__ void pstaged_consume(const typename Op::Params &p, uint64_t *full, uint64_t *empty,
                                                const typename Op::Tin *buf, int &s, uint32_t &ph, const PUnit &un)
{
    using T = typename Op::Tin;
    constexpr int MH = Op::MH, HY = Op::HY, PX = Op::PX, NIN = Op::NIN, SEGW = PX + 2 * Op::HX;
    const Geom &g = p.g;
    const int S = g.stages, SW = g.sw, HXA = g.hxa;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int nr = un.rows + 2 * HY;
    const size_t row_elems = (size_t)NIN * SW;
    const int xoff = (warp * 32 + lane) * PX;
    const int x0 = un.x0 + xoff;
    typename Op::A acc[MH];
#pragma unroll
    for (int k = 0; k < MH; ++k) Op::zero(acc[k]);
    for (int r0 = 0; r0 < nr; r0 += MH) {
#pragma unroll
        for (int k = 0; k < MH; ++k) {
            const int r = r0 + k;
            if (r < nr) {
                mbar_wait(&full[s], ph);
                const T *rb = buf + (size_t)s * row_elems;
                RawRow<Op> rr;
                const T *srow[NIN];
#pragma unroll
                for (int c = 0; c < NIN; ++c) srow[c] = rb + (size_t)c * SW + HXA + xoff;
                load_row_smem<Op>(srow, rr);
                __syncwarp();
                if (lane == 0) mbar_arrive(&empty[s]);  // the row is in registers: release the slot
                if (++s == S) { s = 0; ph ^= 1; }
                T seg[NIN][SEGW];
                unpack_row<Op>(rr, seg);
                if constexpr ((CK & (CK_L | CK_R)) != 0) {
                    if (consumer_fix(g, PX)) staged_edge_fix<Op, CK>(g, x0, seg, p.cval);
                }
                typename Op::H hs;
                Op::hrow(p, seg, hs);
                Op::template vacc<true>(p, 0, hs, acc[k]);
#pragma unroll
                for (int j = 1; j < MH; ++j) {
                    if (!Op::row_used(j)) continue;
                    Op::template vacc<false>(p, j, hs, acc[(k - j + MH) % MH]);
                }
                const int o = r - (MH - 1);
                if (o >= 0) Op::template store<CK & CK_R>(p, acc[(k + 1) % MH], x0, un.y0 + o);
            }
        }
    }
}

template <class Op, int MODE>
__device__ __forceinline__ void pstaged_producer_loop(const typename Op::Params &p, uint64_t *full, uint64_t *empty,
                                                   int4 *meta, typename Op::Tin *buf)
{
    const Geom &g = p.g;
    const int lane = threadIdx.x & 31;
    int s = 0;
    uint32_t ph = 0;
    long long nfill = 0;
    unsigned int *ctr = g.sched;
    // claims run one unit ahead: the atomic of unit i+1 is in flight while unit i's rows
    // are issued, so its L2 round trip does not stall the ring
    unsigned int nxt = 0;
    if (lane == 0) nxt = atomicAdd(ctr, 1u);
    for (;;) {
        int u = (int)__shfl_sync(0xffffffffu, nxt, 0);
        if (u >= g.nunits) break;
        if (lane == 0) nxt = atomicAdd(ctr, 1u);
        const PUnit un = punit_of(g, u);
        switch (un.rg) {
        case RG_TL: pstaged_produce<Op, MODE, region_checks(RG_TL)>(p, full, empty, meta, buf, s, ph, nfill, u, un); break;
        case RG_TR: pstaged_produce<Op, MODE, region_checks(RG_TR)>(p, full, empty, meta, buf, s, ph, nfill, u, un); break;
        case RG_T: pstaged_produce<Op, MODE, region_checks(RG_T)>(p, full, empty, meta, buf, s, ph, nfill, u, un); break;
        case RG_BL: pstaged_produce<Op, MODE, region_checks(RG_BL)>(p, full, empty, meta, buf, s, ph, nfill, u, un); break;
        case RG_BR: pstaged_produce<Op, MODE, region_checks(RG_BR)>(p, full, empty, meta, buf, s, ph, nfill, u, un); break;
        case RG_B: pstaged_produce<Op, MODE, region_checks(RG_B)>(p, full, empty, meta, buf, s, ph, nfill, u, un); break;
        case RG_R: pstaged_produce<Op, MODE, region_checks(RG_R)>(p, full, empty, meta, buf, s, ph, nfill, u, un); break;
        case RG_L: pstaged_produce<Op, MODE, region_checks(RG_L)>(p, full, empty, meta, buf, s, ph, nfill, u, un); break;
        default: pstaged_produce<Op, MODE, 0>(p, full, empty, meta, buf, s, ph, nfill, u, un); break;
        }
    }
    // sentinel slot: the consumers stop
    if (nfill >= g.stages) mbar_wait(&empty[s], ph ^ 1);
    if (lane == 0) meta[s] = make_int4(-1, 0, 0, 0);
    cp_async_mbar_arrive_noinc(&full[s]);
    if (lane == 0) mbar_arrive(&full[s]);
    // the last CTA to finish claiming resets the scheduler for the next launch
    if (lane == 0) {
        __threadfence();
        if (atomicAdd(ctr + 1, 1u) == gridDim.x - 1) {
            atomicExch(ctr, 0u);
            atomicExch(ctr + 1, 0u);
        }
    }
}

template <class Op>
__device__ __forceinline__ void pstaged_consumer_loop(const typename Op::Params &p, uint64_t *full, uint64_t *empty,
                                                   const int4 *meta, const typename Op::Tin *buf)
{
    const Geom &g = p.g;
    int s = 0;
    uint32_t ph = 0;
    for (;;) {
        mbar_wait(&full[s], ph);
        const int4 m = meta[s];
        if (m.x < 0) break;
        const PUnit un = punit_of(g, m.x);
        switch (un.rg) {
        case RG_TL: pstaged_consume<Op, region_checks(RG_TL)>(p, full, empty, buf, s, ph, un); break;
        case RG_TR: pstaged_consume<Op, region_checks(RG_TR)>(p, full, empty, buf, s, ph, un); break;
        case RG_T: pstaged_consume<Op, region_checks(RG_T)>(p, full, empty, buf, s, ph, un); break;
        case RG_BL: pstaged_consume<Op, region_checks(RG_BL)>(p, full, empty, buf, s, ph, un); break;
        case RG_BR: pstaged_consume<Op, region_checks(RG_BR)>(p, full, empty, buf, s, ph, un); break;
        case RG_B: pstaged_consume<Op, region_checks(RG_B)>(p, full, empty, buf, s, ph, un); break;
        case RG_R: pstaged_consume<Op, region_checks(RG_R)>(p, full, empty, buf, s, ph, un); break;
        case RG_L: pstaged_consume<Op, region_checks(RG_L)>(p, full, empty, buf, s, ph, un); break;
        default: pstaged_consume<Op, 0>(p, full, empty, buf, s, ph, un); break;
        }
    }
}

// The persistent TMA-staged fat kernel.  blockDim.x = 32 * (nwc + 1).
template <class Op>
__global__ void __launch_bounds__(32 * (kPMaxComputeWarps + 1)) k_pstaged(const __grid_constant__ typename Op::Params p)
{
    extern __shared__ __align__(128) unsigned char smem[];
    const Geom &g = p.g;
    uint64_t *full = reinterpret_cast<uint64_t *>(smem);
    uint64_t *empty = full + kPMaxStages;
    int4 *meta = reinterpret_cast<int4 *>(smem + 2 * kPMaxStages * sizeof(uint64_t));
    using T = typename Op::Tin;
    T *buf = reinterpret_cast<T *>(smem + kPHeaderBytes);
    const int warp = threadIdx.x >> 5;
    if (threadIdx.x == 0) {
        for (int s = 0; s < g.stages; ++s) {
            mbar_init(&full[s], 33);   // 32 producer lanes (cp.async arrive) + lane 0 (expect_tx)
            mbar_init(&empty[s], g.nwc);
        }
        fence_mbar_init();
    }
    __syncthreads();
    pdl_launch_dependents();
    pdl_wait();  // the prologue above overlaps the previous kernel's tail (PDL)
    if (warp == g.nwc) {
        switch (g.mode) {  // the border pattern is a runtime parameter (producer code only)
        case CLAMP: pstaged_producer_loop<Op, CLAMP>(p, full, empty, meta, buf); break;
        case MIRROR: pstaged_producer_loop<Op, MIRROR>(p, full, empty, meta, buf); break;
        case REPEAT: pstaged_producer_loop<Op, REPEAT>(p, full, empty, meta, buf); break;
        default: pstaged_producer_loop<Op, CONSTANT>(p, full, empty, meta, buf); break;
        }
        return;
    }
    pstaged_consumer_loop<Op>(p, full, empty, meta, buf);
}

}  // namespace ispk
