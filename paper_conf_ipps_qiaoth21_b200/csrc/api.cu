// api.cu -- the C ABI (include/isp.h): validation, the region planner and analytic
// model (Eqs. 2-10), variant selection ("isp+m") and kernel launch.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <functional>
#include <mutex>
#include <unordered_map>
#include <vector>

#include "../../include/isp.h"
#include "internal.h"
#include "kernels.h"

using namespace ispk;

namespace {

thread_local char g_err[512] = "";
thread_local isp_plan_info g_last_plan{};
// the last kRecent resolved plans of this thread (multi-launch calls: Night, strips)
constexpr int kRecent = 16;
thread_local isp_plan_info g_recent[kRecent];
thread_local long long g_n_plans = 0;
int g_override_wx = 0, g_override_ty = 0;

// Rows of the strips holding the image's top / bottom border in a balanced split, in
// 1/256 of an interior strip (0 = uniform); ISP_EDGE_W overrides.
constexpr int kEdgeW = 64;
int edge_w_setting()
{
    const char *e = getenv("ISP_EDGE_W");
    return e ? std::max(0, atoi(e)) : kEdgeW;
}

}  // namespace

isp_status_t ispi_fail(isp_status_t s, const char *fmt, ...)
{
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(g_err, sizeof(g_err), fmt, ap);
    va_end(ap);
    return s;
}

namespace {
#define fail ispi_fail

isp_status_t cuda_status(cudaError_t e, const char *what)
{
    if (e == cudaSuccess) return ISP_OK;
    if (e == cudaErrorNotSupported) return fail(ISP_EUNSUPPORTED, "%s: not built for this window", what);
    return fail(ISP_ECUDA, "%s: %s", what, cudaGetErrorString(e));
}

long long floor_div(long long a, long long b) { return a >= 0 ? a / b : -((-a + b - 1) / b); }
long long ceil_div(long long a, long long b) { return -floor_div(-a, b); }

bool ranges_overlap(const void *a, size_t abytes, const void *b, size_t bbytes)
{
    const char *pa = (const char *)a, *pb = (const char *)b;
    return pa < pb + bbytes && pb < pa + abytes;
}

size_t img_bytes(int w, int h, int pitch, size_t es) { return ((size_t)(h - 1) * pitch + w) * es; }

isp_status_t check_geom(int w, int h, int pitch, int out_pitch, int mw, int mh, int mode)
{
    if (w < 1 || h < 1) return fail(ISP_EINVAL, "image size %dx%d", w, h);
    if (pitch < w || out_pitch < w) return fail(ISP_EINVAL, "pitch %d / out_pitch %d < width %d", pitch, out_pitch, w);
    if (mw < 1 || mh < 1 || mw > 31 || mh > 31 || (mw % 2) == 0 || (mh % 2) == 0)
        return fail(ISP_EINVAL, "window %dx%d must be odd and in [1,31] (reading A8)", mw, mh);
    if (mode < 0 || mode > 3) return fail(ISP_EINVAL, "border mode %d", mode);
    return ISP_OK;
}

// ---------------------------------------------------------------------------------
// Planner: Eq. (2) (reading A2), Eq. (7), Listing 5 warp bounds (A22), Eq. (8) (A17).
// ---------------------------------------------------------------------------------
struct Plan {
    int px, wx, ty, tile_w, warp_w;
    int nx, ny;
    int bh_l, bh_r, bh_t, bh_b, w_l, w_r;
    int edge_w;  // balanced split: weight of the image's first / last strip (x 1/256)
    bool degenerate;
    // pixel rows of the block rows in the T class (by < BH_T), the middle class and the
    // B class (by >= BH_B): uniform tiles -> count * ty (Eq. 5 as printed, reading A25);
    // balanced split -> the real rows of those block rows
    long long rows_t, rows_m, rows_b;
};

int g_num_sms = 0;

int num_sms()
{
    if (g_num_sms <= 0) {
        int dev = 0, n = 0;
        if (cudaGetDevice(&dev) == cudaSuccess && cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev) ==
                                                      cudaSuccess && n > 0)
            g_num_sms = n;
        else {
            cudaGetLastError();
            g_num_sms = 148;  // B200 (no device visible: pure-host planning)
        }
    }
    return g_num_sms;
}

constexpr int kMinRowsPerBlock = 8;
constexpr int kStreamTileRows = 16;

// blocks_per_sm: resident blocks of the kernel that will run (occupancy API); 0 = 8.
// hx, hy: reach of the window to the left / top of the anchor; hxr, hyb (default hx, hy):
// to the right / bottom -- the non-zero footprint of a sparse mask (reading A31).
Plan make_plan(int w, int h, int hx, int hy, int px, int tile_w_req, int tile_h_req, int warp_w_req,
               const RowRange *rr = nullptr, int blocks_per_sm = 0, int hxr = -1, int hyb = -1)
{
    if (hxr < 0) hxr = hx;
    if (hyb < 0) hyb = hy;
    const RowRange whole{0, h, h, 1, 1};
    if (!rr) rr = &whole;
    Plan p{};
    p.px = px;
    const int warp_w = warp_w_req > 0 ? warp_w_req : 32 * px;
    int wx;
    if (tile_w_req > 0) {
        wx = std::max(1, tile_w_req / warp_w);
    } else if (g_override_wx > 0) {
        wx = g_override_wx;
    } else {
        wx = (int)std::min<long long>(4, std::max<long long>(1, ceil_div(w, warp_w)));
    }
    p.wx = wx;
    p.warp_w = warp_w;
    p.tile_w = wx * warp_w;
    p.nx = (int)ceil_div(w, p.tile_w);
    const int nr = rr->nrows;
    const int ty_req = tile_h_req > 0 ? tile_h_req : g_override_ty;
    if (ty_req > 0) {
        // uniform tiles of ty rows: Eq. (2) verbatim in y
        p.ty = ty_req;
        p.ny = (int)ceil_div(nr, p.ty);
    } else {
        // balanced split: one wave of resident blocks, >= kMinRowsPerBlock rows each
        const long long slots = (long long)num_sms() * (blocks_per_sm > 0 ? blocks_per_sm : 8);
        long long nby = std::max<long long>(1, slots / p.nx);
        nby = std::min<long long>(nby, std::max(1, nr / kMinRowsPerBlock));
        p.ty = 0;
        p.ny = (int)nby;
    }
    p.bh_l = (int)ceil_div(hx, p.tile_w);
    p.bh_r = (int)floor_div(w - hxr, p.tile_w);
    p.w_l = (int)ceil_div(hx, warp_w);
    p.w_r = (int)floor_div(w - hxr, warp_w);
    // Eq. (2) in y, relative to the launch's first row oy0; only real image edges count.
    // a peer strip's edges are region edges as well (rows beyond them live in another
    // buffer): top edge at own_y0, bottom edge at own_y1 (reading of SURVEY 8(f) N4)
    const bool pt = rr->peer && !rr->t_real, pb = rr->peer && !rr->b_real;
    const long long top_edge = rr->t_real ? 0 : rr->own_y0, bot_edge = rr->b_real ? h : rr->own_y1;
    if (p.ty > 0) {
        p.bh_t = (rr->t_real || pt) ? (int)std::max<long long>(0, ceil_div(hy - (rr->oy0 - top_edge), p.ty)) : 0;
        const long long safe_end = (rr->b_real || pb) ? std::min<long long>(rr->oy0 + nr, bot_edge - hyb)
                                                      : rr->oy0 + nr;
        p.bh_b = (int)floor_div(safe_end - rr->oy0, p.ty);
    } else {
        // same definition on the balanced split: first block row whose reads stay >= 0,
        // first block row whose reads reach past the image bottom
        // (block_rows in isp_core.cuh: border strips weighted by edge_w / 256)
        p.edge_w = p.ny > 2 ? edge_w_setting() : 0;
        const long long ft = rr->t_real ? p.edge_w : 256, fb = rr->b_real ? p.edge_w : 256;
        const long long W = ft + fb + 256ll * (p.ny - 2);
        auto y0_of = [&](long long by) {
            if (p.edge_w <= 0) return rr->oy0 + (by * nr) / p.ny;
            const long long c = by == 0 ? 0 : by == p.ny ? W : ft + 256ll * (by - 1);
            return rr->oy0 + (c * nr) / W;
        };
        int bt = 0;
        if (rr->t_real || pt)
            while (bt < p.ny && y0_of(bt) - hy < top_edge) ++bt;
        int bb = p.ny;
        if (rr->b_real || pb)
            while (bb > 0 && y0_of(bb) + hyb > bot_edge) --bb;   // y0_of(bb) = end of block bb-1
        p.bh_t = bt;
        p.bh_b = bb;
        if (bt <= bb) {
            p.rows_t = y0_of(bt) - y0_of(0);
            p.rows_m = y0_of(bb) - y0_of(bt);
            p.rows_b = y0_of(p.ny) - y0_of(bb);
        }
    }
    if (p.ty > 0 && p.bh_t <= p.bh_b) {
        p.rows_t = (long long)p.bh_t * p.ty;
        p.rows_m = (long long)(p.bh_b - p.bh_t) * p.ty;
        p.rows_b = (long long)(p.ny - p.bh_b) * p.ty;
    }
    p.degenerate = p.bh_l > p.bh_r || p.bh_t > p.bh_b;
    return p;
}

void n_block(const Plan &p, long long nb[9])
{
    const long long L = p.bh_l, R = p.bh_r, T = p.bh_t, B = p.bh_b, NX = p.nx, NY = p.ny;
    nb[0] = L * T;                 // TL
    nb[1] = (NX - R) * T;          // TR
    nb[2] = (R - L) * T;           // T
    nb[3] = L * (NY - B);          // BL
    nb[4] = (NX - R) * (NY - B);   // BR
    nb[5] = (R - L) * (NY - B);    // B
    nb[6] = (NX - R) * (B - T);    // R
    nb[7] = L * (B - T);           // L
    long long s = 0;
    for (int k = 0; k < 8; ++k) s += nb[k];
    nb[8] = NX * NY - s;           // Body, Eq. (8b)
}

// Listing 3 compares per region under short-circuit evaluation (A18), Eq. (4) order.
const int kNSwitch[9] = {2, 3, 3, 6, 8, 8, 8, 9, 8};

// Eqs. (3)-(6), (9), (10).
// Eqs. (3)-(6), (9), (10).  h: rows of the launch's iteration space (the whole image, or a
// strip's rows).  Regions are products of a column class (L: bx < BH_L, middle, R) and a
// row class (T, middle, B); the pixels of region r are ncols(r) * tile_w * rows(class),
// which is n_block(r) * tx * ty for uniform tiles (Eq. 5) and the real block rows for the
// balanced split.  Forms (reading A14 / A21):
//   T (0): n(r) = n_switch(r) threads n_block(r) + n_region(r) m n pixels(r)
//   P (1): n(r) = (n_switch(r) + n_region(r)) m n pixels(r)                     (as printed)
//   S (2): staged kernels, checks paid per STAGED element E(r) = ncols(r) (tx + 2 hx)
//          (rows(class) + 2 hy nblockrows(class)):
//          n(r) = n_switch(r) threads n_block(r) + n_chk(r) n_check E(r) + n_kernel m n pixels(r)
void model(const Plan &p, int w, int h, int mw, int mh, const isp_model_params &mp, isp_plan_info &o)
{
    const double m = mw, n = mh, c = mp.n_check, k = mp.n_kernel;
    o.n_naive = (4 * c + k) * m * n * (double)w * h;             // Eq. (3), reading A13
    if (p.degenerate) {
        o.n_isp = INFINITY;
        o.r_reduced = 0;
        o.g = 0;
        return;
    }
    const double threads = 32.0 * p.wx, tx = p.tile_w;
    const double cols[3] = {(double)p.bh_l, (double)(p.bh_r - p.bh_l), (double)(p.nx - p.bh_r)};  // L, mid, R
    const double rows[3] = {(double)p.rows_t, (double)p.rows_m, (double)p.rows_b};                 // T, mid, B
    const double brows[3] = {(double)p.bh_t, (double)(p.bh_b - p.bh_t), (double)(p.ny - p.bh_b)};
    const int hx = mw / 2, hy = mh / 2;
    // region id (Eq. 4 order) of (row class, column class)
    static const int kReg[3][3] = {{RG_TL, RG_T, RG_TR}, {RG_L, RG_BODY, RG_R}, {RG_BL, RG_B, RG_BR}};
    double nisp = 0;
    for (int rc = 0; rc < 3; ++rc)
        for (int cc = 0; cc < 3; ++cc) {
            const int r = kReg[rc][cc];
            const int nchk = (rc != 1) + (cc != 1);                 // Eq. (6), reading A15
            const double nreg = nchk * c + k;
            const double nsw = kNSwitch[r] * mp.ipc_switch;
            const double nb = cols[cc] * brows[rc];
            const double pix = cols[cc] * tx * rows[rc];
            if (mp.form == 1) nisp += (nsw + nreg) * m * n * pix;
            else if (mp.form == 3) {
                // band kernels (reading A34): a checked side costs one check per staged row per
                // thread of the warp (T / B: the row map; L / R: the edge lanes' halo word)
                const double srows = nb > 0 ? rows[rc] + 2.0 * hy * brows[rc] : 0.0;
                nisp += nsw * threads * nb + nchk * c * threads * srows * cols[cc] + k * m * n * pix;
            } else if (mp.form == 2) {
                const double E = cols[cc] * (tx + 2.0 * hx) * (rows[rc] + 2.0 * hy * brows[rc]);
                nisp += nsw * threads * nb + nchk * c * E + k * m * n * pix;
            } else nisp += nsw * threads * nb + nreg * m * n * pix;
        }
    o.n_isp = nisp;
    o.r_reduced = o.n_naive / nisp;                                  // Eq. (9)
    o.g = o.r_reduced * o.o_isp / o.o_naive;                         // Eq. (10)
}

// Resident blocks per SM of a kernel (occupancy API), cached per (kernel, block size).
int blocks_per_sm(const void *fn, int threads, size_t smem = 0)
{
    static std::mutex mu;
    static std::unordered_map<const void *, std::pair<size_t, int>> cache[9];
    if (!fn) return 0;
    const int slot = smem ? 0 : std::min(8, threads / 32);
    {
        std::lock_guard<std::mutex> lk(mu);
        auto it = cache[slot].find(fn);
        if (it != cache[slot].end() && it->second.first == smem) return it->second.second;
    }
    int nb = 0;
    if (smem > 48 * 1024 && cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) !=
                                cudaSuccess)
        cudaGetLastError();
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, fn, threads, smem) != cudaSuccess) {
        cudaGetLastError();
        nb = 0;
    }
    std::lock_guard<std::mutex> lk(mu);
    cache[slot][fn] = {smem, nb};
    return nb;
}

// Theoretical occupancy O (reading A20): resident warps / 64 warps per SM on sm_100.
double occupancy_of(int nb, int threads) { return std::min(1.0, nb * (threads / 32.0) / 64.0); }

enum Family { F_CONV_F32 = 0, F_SEP_F32 = 1, F_U8 = 2, F_SOBEL = 3, F_LAPLACE = 4, F_HARRIS = 5,
              F_BILATERAL = 6, F_ATROUS = 7 };

int family_px(int fam, bool direct)
{
    if (direct) return PX_DIRECT;
    switch (fam) {
    case F_U8: return PX_U8;
    case F_SOBEL: return kPxSobel;
    case F_LAPLACE: return kPxLaplace;
    case F_HARRIS: return PX_I16;
    default: return PX_F32;
    }
}

// Model constants (reading A19), calibrated on B200 from ncu instruction counts
// (profiles/r02_counters.json, tools/ncu_counters.py): per family and border mode, with I
// = smsp__thread_inst_executed of one 4096^2 (Bilateral 2048^2) launch of px pixels,
//   n_kernel = I_isp / (m n px)              (the ISP launch is essentially its Body)
//   n_check  = (I_naive - I_isp) / (4 m n px)
// i.e. instructions per tap of the computation and per border check per tap.  Families
// in enum order F_CONV_F32 .. F_ATROUS; modes Clamp, Mirror, Repeat, Constant.
const double kCalib[8][4][2] = {
    {{0.1813, 1.7136}, {0.2368, 1.7221}, {0.5511, 1.6320}, {0.1120, 1.6949}},  // F_CONV_F32   (5x5 2-D)
    {{0.1775, 0.8283}, {0.2475, 0.7370}, {0.5045, 0.8338}, {0.1129, 0.7146}},  // F_SEP_F32    (cfg2 5x5)
    {{0.1534, 1.2677}, {0.2122, 1.2649}, {0.5123, 1.2502}, {0.2000, 1.2739}},  // F_U8         (5x5 Gaussian)
    {{0.4532, 3.8122}, {0.5306, 3.8202}, {1.1165, 3.8433}, {0.4094, 3.8157}},  // F_SOBEL
    {{0.1586, 0.9486}, {0.2288, 0.9393}, {0.4854, 0.9581}, {0.2037, 0.9316}},  // F_LAPLACE
    {{0.7511, 6.3915}, {0.8680, 6.3961}, {2.2974, 6.4217}, {0.4643, 6.4138}},  // F_HARRIS
    {{0.1995, 7.0678}, {0.3360, 7.1017}, {2.7004, 7.6321}, {0.6625, 7.2551}},  // F_BILATERAL  (13x13)
    {{0.5936, 2.7106}, {0.6870, 2.7154}, {2.5672, 2.8571}, {0.6184, 2.7451}},  // F_ATROUS     (d = 2)
};

void defaults(int fam, int mode, isp_model_params &mp)
{
    const int f = std::max(0, std::min(7, fam)), m = mode & 3;
    mp.n_check = kCalib[f][m][0];
    mp.n_kernel = kCalib[f][m][1];
    mp.ipc_switch = 2.0;   // ISETP + BRA per Listing-3 compare (A18)
    mp.o_naive = -1;
    mp.o_isp = -1;
    mp.form = 0;
}

using KfnFn = const void *(*)(const Desc &);
using RunFn = cudaError_t (*)(const Desc &);

// TMA-staged family geometry (isp_staged.cuh): 4 compute warps per CTA, tile width
// 128*PX, halo rounded up to 16 B (HXA) and Eq. (2)'s x bounds taken with HXA and the
// 16-B aligned width w_al, so every Body CTA's bulk copies are in bounds (A21).
struct StagedGeom {
    int hxa, w_al, sw, stages, rs, tail;
    size_t smem;
};

// Persistent TMA-staged kernel (isp_pstaged.cuh) knobs: compute warps per CTA, unit
// height CH, ring bytes per CTA, CTAs per SM.
struct PKnobs {
    bool on;
    int nwc, ch, ring_kb, ctas;
};

int env_int(const char *name, int dflt, int lo, int hi)
{
    const char *e = getenv(name);
    if (!e) return dflt;
    return std::max(lo, std::min(hi, atoi(e)));
}

PKnobs pknobs()
{
    PKnobs k;
    // the one-wave static split is the default (measured faster on B200);
    // ISP_TMA_PERSIST=1 selects the persistent dynamic-unit kernel
    k.on = env_int("ISP_TMA_PERSIST", 0, 0, 1) == 1 && env_int("ISP_TMA_STATIC", 0, 0, 1) == 0;
    k.nwc = env_int("ISP_P_NWC", 8, 1, kPMaxComputeWarps);   // best measured: 8 warps x 4 CTAs/SM
    k.ch = env_int("ISP_P_CH", 16, 1, 4096);
    k.ring_kb = env_int("ISP_P_RING_KB", 48, 4, 220);
    k.ctas = env_int("ISP_P_CTAS", 4, 1, 8);
    return k;
}

StagedGeom staged_geom(int w, int hx, int hy, int px, int esz, int nin, int nwc = STAGED_WARPS,
                       bool persistent = false, int ring_kb = 0)
{
    StagedGeom sg{};
    const int tw = nwc * 32 * px;
    // halo rounded up to a whole number of 32-B L2 sectors: the bulk copies then start
    // and end on sector boundaries (16-B-aligned copies straddle sectors)
    int align = 32;
    if (const char *e = getenv("ISP_HALO_ALIGN")) align = std::max(16, atoi(e));
    sg.hxa = (int)(ceil_div((long long)hx * esz, align) * align / esz);
    sg.w_al = (int)(((long long)w * esz / 16) * 16 / esz);
    sg.sw = tw + 2 * sg.hxa;
    const long long row_bytes = (long long)nin * sg.sw * esz;
    if (persistent) {
        // one row per slot; as many slots as fit the ring budget (>= 4, <= 64)
        sg.rs = 1;
        sg.stages = (int)std::min<long long>(kPMaxStages, std::max<long long>(4, (ring_kb * 1024LL) / row_bytes));
        if (const char *e = getenv("ISP_STAGES")) sg.stages = std::max(2, std::min(kPMaxStages, atoi(e)));
        sg.smem = kPHeaderBytes + (size_t)sg.stages * row_bytes;
        return sg;
    }
    // ring of single-row slots, >= 4 slots / ~8 KB of rows in flight per CTA: measured
    // best on B200 for the one-wave static split
    sg.rs = 1;
    if (const char *e = getenv("ISP_RS")) sg.rs = std::max(1, std::min(16, atoi(e)));
    const long long slot_bytes = row_bytes * sg.rs;
    sg.stages = (int)std::min<long long>(32, std::max<long long>(4, ceil_div(8 * 1024, slot_bytes)));
    if (const char *e = getenv("ISP_STAGES")) sg.stages = std::max(2, std::min(32, atoi(e)));
    sg.tail = 0;   // tail prefetch: rejected
    sg.smem = 512 + (size_t)sg.stages * slot_bytes;
    return sg;
}

void apply_staged_bounds(Plan &p, int w, int px, const StagedGeom &sg, int nwc = STAGED_WARPS)
{
    p.wx = nwc;
    p.warp_w = 32 * px;
    p.tile_w = nwc * 32 * px;
    p.nx = (int)ceil_div(w, p.tile_w);
    p.bh_l = (int)ceil_div(sg.hxa, p.tile_w);
    p.bh_r = (int)floor_div(sg.w_al - sg.hxa, p.tile_w);
    p.w_l = p.bh_l * nwc;
    p.w_r = p.bh_r * nwc;
    p.degenerate = p.bh_l > p.bh_r || p.bh_t > p.bh_b;
}

// Scheduler counter pairs of the persistent staged kernels: one pair per (device,
// stream), 32 B apart, zero between launches (the last CTA of a launch resets its pair).
unsigned int *sched_counter(cudaStream_t st)
{
    static std::mutex mu;
    static std::unordered_map<int, unsigned int *> pools;
    static std::unordered_map<long long, int> slots;
    constexpr int kSlots = 1024;
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) return nullptr;
    std::lock_guard<std::mutex> lk(mu);
    unsigned int *&pool = pools[dev];
    if (!pool) {
        if (cudaMalloc(&pool, kSlots * 32) != cudaSuccess || cudaMemset(pool, 0, kSlots * 32) != cudaSuccess ||
            cudaDeviceSynchronize() != cudaSuccess) {
            cudaGetLastError();
            pool = nullptr;
            return nullptr;
        }
    }
    const long long key = ((long long)dev << 56) ^ (long long)(uintptr_t)st;
    auto it = slots.find(key);
    if (it == slots.end()) it = slots.emplace(key, (int)(slots.size() % kSlots)).first;
    return pool + 8 * it->second;
}

// Diagnostics: per-CTA timestamps of TMA-staged launches (env ISP_CTA_TRACE), 4 words
// per CTA, read back with isp_debug_cta_trace.
constexpr int kTraceCtas = 1 << 16;
unsigned long long *cta_trace_buffer()
{
    static unsigned long long *buf = nullptr;
    if (!buf && cudaMalloc(&buf, sizeof(unsigned long long) * 4 * kTraceCtas) != cudaSuccess) buf = nullptr;
    return buf;
}

// Resolve the variant (AUTO = "isp+m") and launch.  tma_ok: the op has a staged
// kernel and the input rows are 16-B aligned; esz / nin: input element size / count.
isp_status_t resolve_and_launch(Desc &d, int fam, int w, int h, int mw, int mh, int hx, int hy, bool direct,
                                isp_variant_t v, KfnFn kfn, RunFn run, const char *what,
                                const RowRange *rr = nullptr, bool tma_ok = false, int esz = 4, int nin = 1)
{
    if (v < ISP_AUTO || v > ISP_SPLIT)
        return fail(v == ISP_TEX ? ISP_EUNSUPPORTED : ISP_EINVAL, "%s: variant %d%s", what, (int)v,
                    v == ISP_TEX ? " (ISP_TEX: isp_filter_ex only)" : "");
    const int px = family_px(fam, direct);
    if (rr) {
        d.g.oy0 = rr->oy0;
        d.g.y_end = rr->oy0 + rr->nrows;
        d.g.ylim = rr->ylim;
        d.g.t_real = rr->t_real;
        d.g.b_real = rr->b_real;
        d.g.peer = rr->peer;
        d.g.own_y0 = rr->own_y0;
        d.g.own_y1 = rr->own_y1;
        d.g.peer_lo = rr->peer_lo;
        d.g.peer_hi = rr->peer_hi;
    }
    // reaches of the window (left, right, top, bottom): the non-zero footprint of a
    // cropped sparse mask (reading A31), else hx / hy on both sides
    const int rl = d.has_reach ? d.reach[0] : hx, rrx = d.has_reach ? d.reach[1] : hx;
    const int rt = d.has_reach ? d.reach[2] : hy, rb = d.has_reach ? d.reach[3] : hy;
    const Plan p0 = make_plan(w, h, rl, rt, px, 0, 0, 0, rr, 0, rrx, rb);
    const int threads = 32 * p0.wx;
    const bool fits = std::max(rl, rrx) <= w && std::max(rt, rb) <= h;  // one reflection suffices (naive Mirror)
    const int naive_disp = fits ? DISP_NAIVE : DISP_NAIVE_GEN;
    auto fn_of = [&](int disp) {
        Desc q = d;
        q.disp = disp;
        return kfn(q);
    };
    // TMA-staged family: persistent dynamic-unit kernel (default) or the one-wave static
    // split (ISP_TMA_STATIC=1); runtime-window (direct) ops: the shared-memory tiled kernel
    // (isp_direct.cuh k_tile), which needs no alignment
    const PKnobs pk = pknobs();
    const bool persist = !direct && pk.on;
    unsigned int *sched = persist ? sched_counter(d.stream) : nullptr;
    const bool use_p = persist && sched != nullptr;
    const int tma_disp = (!direct && !use_p) ? DISP_TMA_STATIC : DISP_TMA;
    const int nwc = use_p ? pk.nwc : STAGED_WARPS;
    StagedGeom sg = staged_geom(w, hx, hy, px, esz, nin, nwc, use_p, pk.ring_kb);
    if (direct) tma_ok = true;
    tma_ok = tma_ok && fn_of(tma_disp) != nullptr && g_override_wx == 0;
    const int tma_threads = direct ? TILE_THREADS : 32 * (nwc + 1);
    size_t tma_smem = direct ? (size_t)(TILE_PX * 32 + d.mw - 1) * (TILE_H + d.mh - 1) * esz : sg.smem;
    const int nb_naive = blocks_per_sm(fn_of(naive_disp), threads);
    const int nb_stream = blocks_per_sm(fn_of(p0.wx > 1 ? DISP_WARP : DISP_BLOCK), threads);
    int nb_tma = tma_ok ? blocks_per_sm(fn_of(tma_disp), tma_threads, tma_smem) : 0;
    if (const char *e = getenv("ISP_CTAS_PER_SM")) nb_tma = std::min(nb_tma, std::max(1, atoi(e)));
    if (use_p) nb_tma = std::min(nb_tma, pk.ctas);
    if (tma_ok && nb_tma <= 0) tma_ok = false;
    // static split with >= 8 resident CTAs / SM: a 3-slot ring per CTA (~50 KB of rows in
    // flight per SM) measured 3 % faster than 4 on cfg2; fewer resident CTAs keep 4 slots
    // (cfg5 7x7: 4 CTAs / SM, 3 slots measured slower) -- DESIGN.md 7b
    if (tma_ok && !direct && !use_p && nb_tma >= 8 && sg.stages == 4 && sg.rs == 1 && !getenv("ISP_STAGES")) {
        sg.stages = 3;
        sg.smem = 512 + (size_t)3 * nin * sg.sw * esz;
        tma_smem = sg.smem;
    }

    // ISP_SPLIT (ablation of P:L90: one kernel per region instead of the fat kernel) plans
    // like ISP_BLOCK and launches each region's block rectangle separately
    const bool split = v == ISP_SPLIT;
    isp_variant_t chosen = split ? ISP_BLOCK : v;
    if (chosen == ISP_TMA && !tma_ok) chosen = ISP_BLOCK;      // misaligned / not built: streaming
    // AUTO's ISP kernel: TMA-staged for 4-byte pixels; for sub-word pixels (u8, i16) the
    // staged L/R CTAs fix up their halo synchronously, so the streaming Listing-5 kernel
    // is faster there (measured, profiles/r01_suite.json cfg3)
    if (v == ISP_AUTO) chosen = (tma_ok && esz == 4) ? ISP_TMA : (p0.wx > 1 ? ISP_WARP : ISP_BLOCK);
    auto plan_for = [&](isp_variant_t c) {
        if (c == ISP_TMA && direct)  // tiles of TILE_PX*32 x TILE_H, Eq. (2) verbatim
            return make_plan(w, h, rl, rt, px, TILE_PX * 32, TILE_H, TILE_PX * 32, rr, nb_tma, rrx, rb);
        if (c == ISP_TMA) {
            // persistent: uniform tiles of nwc*32*px x CH (Eq. 2 verbatim in y);
            // static: the balanced one-wave row split
            int ch = use_p ? pk.ch : 0;
            if (use_p) {
                // short launches: halve the unit height until every resident CTA gets a
                // unit (load balance) -- also keeps Eq. (2) non-degenerate in y
                const long long nxu = ceil_div(w, (long long)nwc * 32 * px), nrw = rr ? rr->nrows : h;
                while (ch > 1 && nxu * ceil_div(nrw, ch) < (long long)num_sms() * nb_tma) ch /= 2;
            }
            Plan q = make_plan(w, h, hx, hy, px, nwc * 32 * px, ch, 0, rr, nb_tma);
            apply_staged_bounds(q, w, px, sg, nwc);
            return q;
        }
        // streaming / naive kernels: uniform tiles of kStreamTileRows rows (Eq. 2 verbatim);
        // several waves of small blocks hide their load latency best (measured)
        // small images: shorter tiles so the grid still covers the SMs (latency-bound)
        int ty = kStreamTileRows;
        const int nrw = rr ? rr->nrows : h;
        while (ty > 1 && (long long)p0.nx * ceil_div(nrw, ty) < num_sms()) ty /= 2;
        return make_plan(w, h, rl, rt, px, 0, g_override_ty > 0 ? 0 : ty, 0, rr,
                         c == ISP_NAIVE ? nb_naive : nb_stream, rrx, rb);
    };
    // the streaming ISP bodies assume vector-aligned rows (isp_core.cuh load_row):
    // misaligned images run the naive kernel (identical results)
    if (!direct && !d.g.vec_in && (chosen == ISP_BLOCK || chosen == ISP_WARP)) chosen = ISP_NAIVE;
    Plan p = plan_for(chosen);
    isp_plan_info info{};
    const bool isp_degenerate = p.degenerate;
    if (p.degenerate) chosen = ISP_NAIVE;  // A3: Listing 3 cannot express a block needing opposite checks
    if (v == ISP_AUTO && !p.degenerate) {
        isp_model_params mp;
        defaults(fam, d.mode, mp);
        info.o_naive = nb_naive > 0 ? occupancy_of(nb_naive, threads) : 1.0;
        // staged / tiled kernels (TMA): latency is hidden by the staging, not by resident
        // warps, so their occupancy term is the naive kernel's (reading A34)
        info.o_isp = chosen == ISP_TMA ? info.o_naive * std::min(1.0, (double)p.nx * p.ny / num_sms())
                                       : (nb_stream > 0 ? occupancy_of(nb_stream, threads) : 1.0);
        n_block(p, info.n_block);
        if (chosen == ISP_TMA) mp.form = 2;   // staged kernels: checks per staged element (A21)
        model(p, w, rr ? rr->nrows : h, mw, mh, mp, info);
        // Eq. (10): ISP iff G > 1 (reading A20), with the calibrated constants (A19)
        if (!(info.g > 1.0)) chosen = ISP_NAIVE;
    }
    if (chosen == ISP_NAIVE) p = plan_for(ISP_NAIVE);
    d.g.ty = p.ty;
    d.g.bh_l = p.bh_l;
    d.g.bh_r = p.bh_r;
    d.g.bh_t = p.bh_t;
    d.g.bh_b = p.bh_b;
    d.g.w_l = p.w_l;
    d.g.w_r = p.w_r;
    d.g.hxa = sg.hxa;
    d.g.w_al = sg.w_al;
    d.g.sw = sg.sw;
    d.g.stages = sg.stages;
    d.g.rs = sg.rs;
    d.g.tail = sg.tail;
    d.grid = dim3(p.nx, p.ny, 1);
    d.block = dim3(chosen == ISP_TMA ? tma_threads : threads, 1, 1);
    d.smem = chosen == ISP_TMA ? tma_smem : 0;
    if (chosen == ISP_TMA && use_p) {
        const long long nunits = (long long)p.nx * p.ny;
        d.g.nux = p.nx;
        d.g.nwc = nwc;
        d.g.px = px;
        d.g.nunits = (int)nunits;
        d.g.sched = sched;
        d.grid = dim3((unsigned)std::min<long long>(nunits, (long long)num_sms() * nb_tma), 1, 1);
    }
    info.bh_l = p.bh_l; info.bh_r = p.bh_r; info.bh_t = p.bh_t; info.bh_b = p.bh_b;
    info.nx = p.nx; info.ny = p.ny; info.w_l = p.w_l; info.w_r = p.w_r;
    info.degenerate = p.degenerate || isp_degenerate;   // the ISP plan's, when it forced NAIVE
    info.tile_w = p.tile_w; info.tile_h = p.ty > 0 ? p.ty : (int)ceil_div(d.g.y_end - d.g.oy0, p.ny);
    info.warp_w = p.warp_w;
    n_block(p, info.n_block);
    info.choice = chosen;
    d.disp = chosen == ISP_TMA ? tma_disp : chosen == ISP_WARP ? DISP_WARP : chosen == ISP_BLOCK ? DISP_BLOCK
                                                                                               : naive_disp;
    d.g.warp_level = chosen == ISP_WARP;
    d.g.mode = d.mode;
    if (const char *e = getenv("ISP_DEBUG_STAGED")) d.g.dbg = atoi(e);
    if (getenv("ISP_CTA_TRACE")) d.g.trace = cta_trace_buffer();
    d.g.edge_w = p.edge_w;
    if (split && chosen == ISP_BLOCK) {
        info.choice = ISP_SPLIT;
        g_last_plan = info;
        g_recent[g_n_plans++ % kRecent] = info;
        const int cx[4] = {0, p.bh_l, p.bh_r, p.nx}, cy[4] = {0, p.bh_t, p.bh_b, p.ny};
        static const int kReg[3][3] = {{RG_TL, RG_T, RG_TR}, {RG_L, RG_BODY, RG_R}, {RG_BL, RG_B, RG_BR}};
        for (int rc = 0; rc < 3; ++rc)
            for (int cc = 0; cc < 3; ++cc) {
                if (cx[cc + 1] <= cx[cc] || cy[rc + 1] <= cy[rc]) continue;
                Desc q = d;
                q.grid = dim3(cx[cc + 1] - cx[cc], cy[rc + 1] - cy[rc], 1);
                q.g.bx0 = cx[cc];
                q.g.by0 = cy[rc];
                q.g.force_rg = kReg[rc][cc];
                cudaError_t e = run(q);
                if (e == cudaSuccess) e = cudaGetLastError();
                if (e != cudaSuccess) return cuda_status(e, what);
            }
        return ISP_OK;
    }
    g_last_plan = info;
    g_recent[g_n_plans++ % kRecent] = info;
    cudaError_t e = run(d);
    if (e == cudaSuccess) e = cudaGetLastError();
    return cuda_status(e, what);
}

// The tile-staged u8 / i16 kernels (tile_u8.cu) as the ISP_TMA variant of Laplace (which
// = 0) and Harris (1): ISP_TMA runs them when eligible; ISP_AUTO evaluates Eq. (10) for
// them (form S, reading A21, calibrated constants, occupancy from the API) against the
// naive kernel.  Returns false when the caller should take the generic path; when AUTO's
// Eq. (10) rejects the ISP kernel, v becomes ISP_NAIVE (the decision is ISP vs naive, not a
// cascade through other ISP implementations).
// which = 2 / 3: the Laplace / Harris band kernels (band_u8.cu: warp strips x bands of rows);
// 4: the separable f32 band kernel (band_f32.cu); 5: Sobel; 6: separable u8.  The band kernels keep several rows in
// flight per warp, so resident warps do not measure their latency hiding: their occupancy
// term is taken equal to the naive kernel's (reading A34).
bool tile_variant(int which, int fam, int mode, int w, int h, int mw, int mh, isp_variant_t &v, bool ok,
                  const std::function<cudaError_t(int *)> &launch, isp_status_t &st, const char *what)
{
    if (!(v == ISP_TMA || v == ISP_AUTO) || !ok) return false;
    int tw, th;
    if (which == 2) ispi_band_shape(w, h, &tw, &th);
    else if (which == 3) ispi_band_harris_shape(w, h, &tw, &th);
    else if (which == 4) ispi_sep_band_shape(w, h, mw, &tw, &th);
    else if (which == 5) ispi_band_sobel_shape(w, h, &tw, &th);
    else if (which == 6) ispi_sepu8_band_shape(w, h, mw, &tw, &th);
    else ispi_tile_shape(&tw, &th);
    Plan p = make_plan(w, h, mw / 2, mh / 2, 4, tw, th, which >= 2 ? tw : 128);
    isp_plan_info info{};
    n_block(p, info.n_block);
    if (v == ISP_AUTO) {
        isp_model_params mp;
        defaults(fam, mode, mp);
        mp.form = which >= 2 ? 3 : 2;   // band form (A34) / staged form S (A21)
        const int nb = which == 4   ? ispi_sep_band_blocks_per_sm(mw)
                       : which == 5 ? ispi_band_blocks_per_sm(2)
                       : which == 6 ? ispi_sepu8_band_blocks_per_sm(mw)
                       : which >= 2 ? ispi_band_blocks_per_sm(which == 3 ? 1 : 0)
                                    : ispi_tile_blocks_per_sm(which);
        info.o_naive = 0.5;   // the naive streaming kernel (64 regs x 128 threads: 8 blocks / SM)
        // band kernels (A34): the naive kernel's occupancy on the SMs the launch reaches
        const double reach = std::min(1.0, (double)ceil_div(p.nx, 4) * p.ny / num_sms());
        info.o_isp = which >= 2 ? info.o_naive * reach : occupancy_of(nb > 0 ? nb : 1, 128);
        model(p, w, h, mw, mh, mp, info);
        if (which >= 2 && p.degenerate) {
            // a band kernel runs one-strip / one-band images too (its edge warps check both
            // sides): form B with every side of every block checked
            const double c = mp.n_check, k = mp.n_kernel, thr = 32.0 * p.wx;
            const double nb = (double)p.nx * p.ny, srows = (double)h + 2.0 * (mh / 2) * p.ny;
            info.n_isp = 8.0 * mp.ipc_switch * thr * nb + 4.0 * c * thr * srows * p.nx + k * mw * mh * (double)w * h;
            info.r_reduced = info.n_naive / info.n_isp;
            info.g = info.r_reduced * info.o_isp / info.o_naive;
        }
        if (!(info.g > 1.0)) {
            v = ISP_NAIVE;
            return false;
        }
    }
    int b[4];
    cudaError_t e = launch(b);
    if (e == cudaSuccess) e = cudaGetLastError();
    info.bh_l = b[0]; info.bh_r = b[1]; info.bh_t = b[2]; info.bh_b = b[3];
    info.nx = p.nx; info.ny = p.ny;
    info.degenerate = 0;
    info.tile_w = tw; info.tile_h = th; info.warp_w = which >= 2 ? tw : 128;
    info.choice = ISP_TMA;
    g_last_plan = info;
    g_recent[g_n_plans++ % kRecent] = info;
    st = cuda_status(e, what);
    return true;
}

Desc base_desc(int w, int h, int pitch, int out_pitch, int mode, isp_stream_t stream)
{
    Desc d{};
    d.g.w = w;
    d.g.h = h;
    d.g.in_pitch = pitch;
    d.g.out_pitch = out_pitch;
    d.g.oy0 = 0;
    d.g.y_end = h;
    d.g.ylim = h;
    d.g.t_real = 1;
    d.g.b_real = 1;
    d.mode = mode;
    d.stream = (cudaStream_t)stream;
    d.g.force_rg = -1;
    return d;
}

bool aligned(const void *p, long long pitch_bytes, int vbytes)
{
    return ((uintptr_t)p % vbytes) == 0 && (pitch_bytes % vbytes) == 0;
}

// exact rank-1 test of a float mask: mask[j][i] == col[j] * row[i]
bool separable_f32(const float *mask, int mw, int mh, std::vector<float> &row, std::vector<float> &col)
{
    int j0 = 0, i0 = 0;
    float best = 0;
    for (int j = 0; j < mh; ++j)
        for (int i = 0; i < mw; ++i)
            if (std::fabs(mask[j * mw + i]) > best) { best = std::fabs(mask[j * mw + i]); j0 = j; i0 = i; }
    if (best == 0) return false;
    row.assign(mask + j0 * mw, mask + j0 * mw + mw);
    col.resize(mh);
    for (int j = 0; j < mh; ++j) col[j] = mask[j * mw + i0] / mask[j0 * mw + i0];
    for (int j = 0; j < mh; ++j)
        for (int i = 0; i < mw; ++i)
            if (std::fabs(col[j] * row[i] - mask[j * mw + i]) > 1e-6f * best) return false;
    return true;
}

long long gcdll(long long a, long long b)
{
    a = a < 0 ? -a : a;
    b = b < 0 ? -b : b;
    while (b) { long long t = a % b; a = b; b = t; }
    return a;
}

// exact integer rank-1 decomposition mask = col (x) row
bool separable_i32(const int32_t *mask, int mw, int mh, std::vector<int> &row, std::vector<int> &col)
{
    int j0 = -1;
    for (int j = 0; j < mh && j0 < 0; ++j)
        for (int i = 0; i < mw; ++i)
            if (mask[j * mw + i] != 0) { j0 = j; break; }
    if (j0 < 0) return false;
    long long g = 0;
    for (int i = 0; i < mw; ++i) g = gcdll(g, mask[j0 * mw + i]);
    row.resize(mw);
    for (int i = 0; i < mw; ++i) row[i] = (int)(mask[j0 * mw + i] / g);
    int i0 = 0;
    while (row[i0] == 0) ++i0;
    col.resize(mh);
    for (int j = 0; j < mh; ++j) {
        if (mask[j * mw + i0] % row[i0] != 0) return false;
        col[j] = mask[j * mw + i0] / row[i0];
    }
    for (int j = 0; j < mh; ++j)
        for (int i = 0; i < mw; ++i)
            if ((long long)col[j] * row[i] != mask[j * mw + i]) return false;
    return true;
}

U8RoundH make_round(int divisor)
{
    U8RoundH r{divisor, -1, 0};
    if (divisor > 0 && (divisor & (divisor - 1)) == 0) {
        int s = 0;
        while ((1 << s) < divisor) ++s;
        r.shift = s;
        r.half = divisor >> 1;
    }
    return r;
}

}  // namespace

// =====================================================================================
extern "C" {

const char *isp_status_string(isp_status_t s)
{
    switch (s) {
    case ISP_OK: return "ISP_OK";
    case ISP_EINVAL: return "ISP_EINVAL";
    case ISP_EUNSUPPORTED: return "ISP_EUNSUPPORTED";
    case ISP_EALIAS: return "ISP_EALIAS";
    case ISP_ECUDA: return "ISP_ECUDA";
    case ISP_ENCCL: return "ISP_ENCCL";
    }
    return "ISP_?";
}

const char *isp_last_error(void) { return g_err; }
int isp_version(void) { return 1; }

/* Diagnostics (not part of the contract): copy the per-CTA trace of the last TMA-staged
 * launches made with ISP_CTA_TRACE set (n CTAs x {smid|region<<16|by<<32|bx<<48, t0, t1, 0}). */
int isp_debug_cta_trace(unsigned long long *host, int n)
{
    unsigned long long *b = cta_trace_buffer();
    if (!b || n < 0 || n > kTraceCtas) return ISP_EINVAL;
    return cudaMemcpy(host, b, sizeof(unsigned long long) * 4 * (size_t)n, cudaMemcpyDeviceToHost) == cudaSuccess
               ? ISP_OK : ISP_ECUDA;
}

isp_status_t isp_last_plan(isp_plan_info *out)
{
    if (!out) return fail(ISP_EINVAL, "null output");
    *out = g_last_plan;
    return ISP_OK;
}

int isp_recent_plans(isp_plan_info *out, int n)
{
    if (!out || n <= 0) return 0;
    const int avail = (int)std::min<long long>(g_n_plans, kRecent);
    const int k = std::min(n, avail);
    for (int i = 0; i < k; ++i) out[i] = g_recent[(g_n_plans - k + i) % kRecent];  // oldest first
    return k;
}

void isp_clear_plans(void)
{
    g_n_plans = 0;
    g_last_plan = isp_plan_info{};
}

// Launch-shape override for tuning sweeps (0 = planner default).  Not thread-safe.
isp_status_t isp_set_launch_override(int warps_x, int tile_h)
{
    if (warps_x < 0 || warps_x > 8 || tile_h < 0 || tile_h > 4096) return fail(ISP_EINVAL, "override");
    g_override_wx = warps_x;
    g_override_ty = tile_h;
    return ISP_OK;
}

}  // extern "C"

// ---------------------------------------------------------------------------------
// Sparse masks (the paper's future work), reading A31: a mask
// with all-zero edge rows / columns is cropped to its non-zero footprint.  Zero taps add
// exactly 0 (finite images), so the cropped window computes the same bits; the ISP
// bounds (Eq. 2) then follow the footprint's reach on each side instead of the bounding
// window.  A footprint that is still a centred odd 3/5/7 square runs the compiled
// kernels; any other footprint runs the direct family with its anchor (ax, ay).
// ---------------------------------------------------------------------------------
struct Crop {
    bool cropped = false;
    int mw, mh, ax, ay;     // cropped window and anchor
    int reach[4];           // L, R, T, B (clamped at 0: partial tiles stay in R / B, A10)
    bool centred() const { return ax == mw - 1 - ax && ay == mh - 1 - ay; }
};

template <class M>
Crop crop_mask(const M *mask, int mw, int mh, std::vector<M> &out)
{
    Crop c;
    c.mw = mw;
    c.mh = mh;
    c.ax = mw / 2;
    c.ay = mh / 2;
    int i0 = mw, i1 = -1, j0 = mh, j1 = -1;
    for (int j = 0; j < mh; ++j)
        for (int i = 0; i < mw; ++i)
            if (mask[j * mw + i] != M(0)) {
                i0 = std::min(i0, i); i1 = std::max(i1, i);
                j0 = std::min(j0, j); j1 = std::max(j1, j);
            }
    if (i1 < 0) { i0 = i1 = mw / 2; j0 = j1 = mh / 2; }     // all zero: the centre tap (weight 0)
    c.reach[0] = std::max(0, mw / 2 - i0);
    c.reach[1] = std::max(0, i1 - mw / 2);
    c.reach[2] = std::max(0, mh / 2 - j0);
    c.reach[3] = std::max(0, j1 - mh / 2);
    if (i0 == 0 && i1 == mw - 1 && j0 == 0 && j1 == mh - 1) return c;
    c.cropped = true;
    c.mw = i1 - i0 + 1;
    c.mh = j1 - j0 + 1;
    c.ax = mw / 2 - i0;
    c.ay = mh / 2 - j0;
    out.resize((size_t)c.mw * c.mh);
    for (int j = 0; j < c.mh; ++j)
        for (int i = 0; i < c.mw; ++i) out[(size_t)j * c.mw + i] = mask[(j + j0) * mw + i + i0];
    return c;
}

bool compiled_window(int mw, int mh) { return mw == mh && (mw == 3 || mw == 5 || mw == 7); }

// Internal row-range entry points (multi-GPU strips, shard.cu).  `img` is addressed
// with global rows; `out` points at the output row rr->oy0.
isp_status_t ispi_filter_f32(const float *img, int w, int h, int pitch, const float *mask, int mw, int mh,
                             int border_mode, float const_val, float *out, int out_pitch, isp_variant_t variant,
                             isp_stream_t stream, const RowRange *rr)
{
    isp_status_t s = check_geom(w, h, pitch, out_pitch, mw, mh, border_mode);
    if (s != ISP_OK) return s;
    if (!img || !out || !mask) return fail(ISP_EINVAL, "null pointer");
    if (!rr && ranges_overlap(img, img_bytes(w, h, pitch, 4), out, img_bytes(w, h, out_pitch, 4)))
        return fail(ISP_EALIAS, "input and output overlap");
    if (variant == ISP_TEX) {   // ablation: texture-hardware border handling (texture.cu)
        if (rr) return fail(ISP_EUNSUPPORTED, "ISP_TEX: row ranges (strips) not supported");
        return ispi_filter_tex_f32(img, w, h, pitch, mask, mw, mh, border_mode, const_val, out, out_pitch, stream);
    }
    Desc d = base_desc(w, h, pitch, out_pitch, border_mode, stream);
    d.in0 = img;
    d.out0 = out;
    d.cval_f = const_val;
    d.mw = mw;
    d.mh = mh;
    d.g.vec_in = aligned(img, (long long)pitch * 4, 16);
    d.g.vec_out = aligned(out, (long long)out_pitch * 4, 16);
    std::vector<float> cm;
    const Crop cr = crop_mask(mask, mw, mh, cm);
    if (cr.cropped) {   // sparse mask: its non-zero footprint (reading A31)
        if (cr.centred() && compiled_window(cr.mw, cr.mh))
            return ispi_filter_f32(img, w, h, pitch, cm.data(), cr.mw, cr.mh, border_mode, const_val, out, out_pitch,
                                   variant, stream, rr);
        d.mw = cr.mw;
        d.mh = cr.mh;
        d.ax = cr.ax;
        d.ay = cr.ay;
        std::memcpy(d.reach, cr.reach, sizeof(d.reach));
        d.has_reach = 1;
        d.maskf = cm.data();
        return resolve_and_launch(d, F_CONV_F32, w, h, cr.mw, cr.mh, cr.reach[0], cr.reach[2], true, variant,
                                  kfn_dconv_f32, run_dconv_f32, "isp_filter(sparse mask)", rr);
    }
    d.ax = mw / 2;
    d.ay = mh / 2;
    std::vector<float> row, col;
    if (compiled_window(mw, mh)) {
        if (separable_f32(mask, mw, mh, row, col)) {
            d.rowf = row.data();
            d.colf = col.data();
            // ISP_TMA / AUTO: the warp-strip band kernel (band_f32.cu; whole images and strips)
            isp_status_t ts;
            if (!getenv("ISP_F32_STAGED") &&
                tile_variant(4, F_SEP_F32, border_mode, w, rr ? rr->nrows : h, mw, mh, variant,
                             ispi_sep_band_ok(img, w, rr ? rr->nrows : h, pitch, out, out_pitch, mw, mh),
                             [&](int *b) { return ispi_sep_band(img, w, h, pitch, row.data(), col.data(), mw,
                                                               border_mode, const_val, out, out_pitch,
                                                               (cudaStream_t)stream, b, rr); },
                             ts, "isp_filter(separable band)"))
                return ts;
            return resolve_and_launch(d, F_SEP_F32, w, h, mw, mh, mw / 2, mh / 2, false, variant, kfn_sep_f32,
                                      run_sep_f32, "isp_filter(separable)", rr,
                                      aligned(img, (long long)pitch * 4, 16), 4, 1);
        }
        d.maskf = mask;
        return resolve_and_launch(d, F_CONV_F32, w, h, mw, mh, mw / 2, mh / 2, false, variant, kfn_conv_f32,
                                  run_conv_f32, "isp_filter", rr, aligned(img, (long long)pitch * 4, 16), 4, 1);
    }
    d.maskf = mask;
    return resolve_and_launch(d, F_CONV_F32, w, h, mw, mh, mw / 2, mh / 2, true, variant, kfn_dconv_f32,
                              run_dconv_f32, "isp_filter(direct)", rr);
}

isp_status_t ispi_filter_u8(const uint8_t *img, int w, int h, int pitch, const int32_t *mask, int mw, int mh,
                            int32_t divisor, int border_mode, int const_val, uint8_t *out, int out_pitch,
                            isp_variant_t variant, isp_stream_t stream, const RowRange *rr)
{
    isp_status_t s = check_geom(w, h, pitch, out_pitch, mw, mh, border_mode);
    if (s != ISP_OK) return s;
    if (!img || !out || !mask) return fail(ISP_EINVAL, "null pointer");
    if (divisor <= 0) return fail(ISP_EINVAL, "divisor %d <= 0", divisor);
    if (const_val < 0 || const_val > 255) return fail(ISP_EINVAL, "u8 constant %d not in [0,255]", const_val);
    long long sabs = 0;
    for (int k = 0; k < mw * mh; ++k) sabs += mask[k] < 0 ? -(long long)mask[k] : mask[k];
    if (sabs * 255 + divisor >= (1LL << 30)) return fail(ISP_EINVAL, "mask too large for int32 accumulation");
    if (!rr && ranges_overlap(img, img_bytes(w, h, pitch, 1), out, img_bytes(w, h, out_pitch, 1)))
        return fail(ISP_EALIAS, "input and output overlap");
    Desc d = base_desc(w, h, pitch, out_pitch, border_mode, stream);
    d.in0 = img;
    d.out0 = out;
    d.cval_i = const_val;
    d.mw = mw;
    d.mh = mh;
    d.rnd = make_round(divisor);
    std::vector<int32_t> cm;
    const Crop cr = crop_mask(mask, mw, mh, cm);
    if (cr.cropped) {   // sparse mask: its non-zero footprint (reading A31)
        if (cr.centred() && compiled_window(cr.mw, cr.mh))
            return ispi_filter_u8(img, w, h, pitch, cm.data(), cr.mw, cr.mh, divisor, border_mode, const_val, out,
                                  out_pitch, variant, stream, rr);
        d.mw = cr.mw;
        d.mh = cr.mh;
        d.ax = cr.ax;
        d.ay = cr.ay;
        std::memcpy(d.reach, cr.reach, sizeof(d.reach));
        d.has_reach = 1;
        d.maski = cm.data();
        d.g.vec_in = aligned(img, pitch, 4);
        d.g.vec_out = aligned(out, out_pitch, 4);
        return resolve_and_launch(d, F_U8, w, h, cr.mw, cr.mh, cr.reach[0], cr.reach[2], true, variant,
                                  kfn_dconv_u8, run_dconv_u8, "isp_filter_u8(sparse mask)", rr);
    }
    d.ax = mw / 2;
    d.ay = mh / 2;
    std::vector<int> row, col;
    if (mw == mh && (mw == 3 || mw == 5 || mw == 7)) {
        d.g.vec_in = aligned(img, pitch, 8);
        d.g.vec_out = aligned(out, out_pitch, 8);
        if (separable_i32(mask, mw, mh, row, col)) {
            d.rowi = row.data();
            d.coli = col.data();
            // ISP_TMA / AUTO on whole images: the band kernel (band_u8.cu) for normalised
            // non-negative masks with a power-of-two divisor (the binomial Gaussians)
            isp_status_t ts;
            if (!rr && tile_variant(6, F_U8, border_mode, w, h, mw, mh, variant,
                                    ispi_sepu8_band_ok(img, w, h, pitch, out, out_pitch, mw, row.data(), col.data(),
                                                       divisor),
                                    [&](int *b) { return ispi_sepu8_band(img, w, h, pitch, mw, row.data(), col.data(),
                                                                         divisor, border_mode, const_val, out,
                                                                         out_pitch, (cudaStream_t)stream, b); },
                                    ts, "isp_filter_u8(separable band)"))
                return ts;
            return resolve_and_launch(d, F_U8, w, h, mw, mh, mw / 2, mh / 2, false, variant, kfn_sep_u8,
                                      run_sep_u8, "isp_filter_u8(separable)", rr, aligned(img, pitch, 16), 1, 1);
        }
        d.maski = mask;
        return resolve_and_launch(d, F_U8, w, h, mw, mh, mw / 2, mh / 2, false, variant, kfn_conv_u8, run_conv_u8,
                                  "isp_filter_u8", rr, aligned(img, pitch, 16), 1, 1);
    }
    d.maski = mask;
    d.g.vec_in = aligned(img, pitch, 4);
    d.g.vec_out = aligned(out, out_pitch, 4);
    return resolve_and_launch(d, F_U8, w, h, mw, mh, mw / 2, mh / 2, true, variant, kfn_dconv_u8, run_dconv_u8,
                              "isp_filter_u8(direct)", rr);
}

extern "C" {

isp_status_t isp_filter_ex(const float *img, int w, int h, int pitch, const float *mask, int mw, int mh,
                           int border_mode, float const_val, float *out, int out_pitch, isp_variant_t variant,
                           isp_stream_t stream)
{
    return ispi_filter_f32(img, w, h, pitch, mask, mw, mh, border_mode, const_val, out, out_pitch, variant, stream,
                           nullptr);
}

isp_status_t isp_filter(const float *img, int w, int h, int pitch, const float *mask, int mw, int mh,
                        int border_mode, float const_val, float *out)
{
    return isp_filter_ex(img, w, h, pitch, mask, mw, mh, border_mode, const_val, out, pitch, ISP_AUTO, nullptr);
}

isp_status_t isp_filter_naive(const float *img, int w, int h, int pitch, const float *mask, int mw, int mh,
                              int border_mode, float const_val, float *out)
{
    return isp_filter_ex(img, w, h, pitch, mask, mw, mh, border_mode, const_val, out, pitch, ISP_NAIVE, nullptr);
}

isp_status_t isp_filter_sep_f32(const float *img, int w, int h, int pitch, const float *row, int mw,
                                const float *col, int mh, int border_mode, float const_val, float *out,
                                int out_pitch, isp_variant_t variant, isp_stream_t stream)
{
    isp_status_t s = check_geom(w, h, pitch, out_pitch, mw, mh, border_mode);
    if (s != ISP_OK) return s;
    if (!img || !out || !row || !col) return fail(ISP_EINVAL, "null pointer");
    if (ranges_overlap(img, img_bytes(w, h, pitch, 4), out, img_bytes(w, h, out_pitch, 4)))
        return fail(ISP_EALIAS, "input and output overlap");
    Desc d = base_desc(w, h, pitch, out_pitch, border_mode, stream);
    d.in0 = img;
    d.out0 = out;
    d.cval_f = const_val;
    d.mw = mw;
    d.mh = mh;
    d.rowf = row;
    d.colf = col;
    d.g.vec_in = aligned(img, (long long)pitch * 4, 16);
    d.g.vec_out = aligned(out, (long long)out_pitch * 4, 16);
    if (mw == mh && (mw == 3 || mw == 5 || mw == 7))
        return resolve_and_launch(d, F_SEP_F32, w, h, mw, mh, mw / 2, mh / 2, false, variant, kfn_sep_f32,
                                  run_sep_f32, "isp_filter_sep_f32", nullptr,
                                  aligned(img, (long long)pitch * 4, 16), 4, 1);
    // other windows: the direct family with the outer-product mask
    std::vector<float> m2((size_t)mw * mh);
    for (int j = 0; j < mh; ++j)
        for (int i = 0; i < mw; ++i) m2[j * mw + i] = col[j] * row[i];
    d.maskf = m2.data();
    d.ax = mw / 2;
    d.ay = mh / 2;
    return resolve_and_launch(d, F_SEP_F32, w, h, mw, mh, mw / 2, mh / 2, true, variant, kfn_dconv_f32,
                              run_dconv_f32, "isp_filter_sep_f32(direct)");
}

isp_status_t isp_filter_u8(const uint8_t *img, int w, int h, int pitch, const int32_t *mask, int mw, int mh,
                           int32_t divisor, int border_mode, int const_val, uint8_t *out, int out_pitch,
                           isp_variant_t variant, isp_stream_t stream)
{
    return ispi_filter_u8(img, w, h, pitch, mask, mw, mh, divisor, border_mode, const_val, out, out_pitch, variant,
                          stream, nullptr);
}

isp_status_t isp_sobel_u8(const uint8_t *img, int w, int h, int pitch, int border_mode, int const_val,
                          int16_t *dx, int16_t *dy, uint8_t *mag, int out_pitch, isp_variant_t variant,
                          isp_stream_t stream)
{
    isp_status_t s = check_geom(w, h, pitch, out_pitch, 3, 3, border_mode);
    if (s != ISP_OK) return s;
    if (!img || (!dx && !dy && !mag)) return fail(ISP_EINVAL, "null pointer");
    if (const_val < 0 || const_val > 255) return fail(ISP_EINVAL, "u8 constant %d not in [0,255]", const_val);
    const size_t ib = img_bytes(w, h, pitch, 1);
    if ((dx && ranges_overlap(img, ib, dx, img_bytes(w, h, out_pitch, 2))) ||
        (dy && ranges_overlap(img, ib, dy, img_bytes(w, h, out_pitch, 2))) ||
        (mag && ranges_overlap(img, ib, mag, img_bytes(w, h, out_pitch, 1))))
        return fail(ISP_EALIAS, "input and output overlap");
    Desc d = base_desc(w, h, pitch, out_pitch, border_mode, stream);
    d.in0 = img;
    d.out0 = dx;
    d.out1 = dy;
    d.out2 = mag;
    d.cval_i = const_val;
    d.mw = d.mh = 3;
    d.g.vec_in = aligned(img, pitch, 8);
    d.g.vec_out = (!dx || aligned(dx, 2LL * out_pitch, 16)) && (!dy || aligned(dy, 2LL * out_pitch, 16)) &&
                  (!mag || aligned(mag, out_pitch, 8));
    // ISP_TMA / AUTO: the band kernel (band_u8.cu) when eligible
    isp_status_t ts;
    if (tile_variant(5, F_SOBEL, border_mode, w, h, 3, 3, variant,
                     ispi_band_sobel_ok(img, w, h, pitch, dx, dy, mag, out_pitch),
                     [&](int *b) { return ispi_sobel_band(img, w, h, pitch, border_mode, const_val, dx, dy, mag, out_pitch,
                                                          (cudaStream_t)stream, b); },
                     ts, "isp_sobel_u8(band)"))
        return ts;
    return resolve_and_launch(d, F_SOBEL, w, h, 3, 3, 1, 1, false, variant, kfn_sobel, run_sobel, "isp_sobel_u8",
                              nullptr, aligned(img, pitch, 16), 1, 1);
}

isp_status_t isp_laplace5_u8(const uint8_t *img, int w, int h, int pitch, int border_mode, int const_val,
                             uint8_t *out, int out_pitch, isp_variant_t variant, isp_stream_t stream)
{
    isp_status_t s = check_geom(w, h, pitch, out_pitch, 5, 5, border_mode);
    if (s != ISP_OK) return s;
    if (!img || !out) return fail(ISP_EINVAL, "null pointer");
    if (const_val < 0 || const_val > 255) return fail(ISP_EINVAL, "u8 constant %d not in [0,255]", const_val);
    if (ranges_overlap(img, img_bytes(w, h, pitch, 1), out, img_bytes(w, h, out_pitch, 1)))
        return fail(ISP_EALIAS, "input and output overlap");
    isp_status_t ts;
    // ISP_TMA / AUTO: the band kernel (band_u8.cu) when eligible, else the tile kernel
    if (tile_variant(2, F_LAPLACE, border_mode, w, h, 5, 5, variant, ispi_band_ok(img, w, h, pitch, out, out_pitch),
                     [&](int *b) { return ispi_laplace_band(img, w, h, pitch, border_mode, const_val, out, out_pitch,
                                                            (cudaStream_t)stream, b); },
                     ts, "isp_laplace5_u8(band)"))
        return ts;
    if (tile_variant(0, F_LAPLACE, border_mode, w, h, 5, 5, variant,
                     ispi_tile_ok(img, nullptr, 1, w, h, pitch, out, out_pitch),
                     [&](int *b) { return ispi_laplace_tile(img, w, h, pitch, border_mode, const_val, out, out_pitch,
                                                            (cudaStream_t)stream, b); },
                     ts, "isp_laplace5_u8(tile)"))
        return ts;
    Desc d = base_desc(w, h, pitch, out_pitch, border_mode, stream);
    d.in0 = img;
    d.out0 = out;
    d.cval_i = const_val;
    d.mw = d.mh = 5;
    d.g.vec_in = aligned(img, pitch, 8);
    d.g.vec_out = aligned(out, out_pitch, 8);
    return resolve_and_launch(d, F_LAPLACE, w, h, 5, 5, 2, 2, false, variant, kfn_laplace5, run_laplace5,
                              "isp_laplace5_u8", nullptr, aligned(img, pitch, 16), 1, 1);
}

isp_status_t isp_harris_u8(const int16_t *dx, const int16_t *dy, int w, int h, int pitch, int border_mode,
                           int const_val, int64_t thr, uint8_t *out, int out_pitch, isp_variant_t variant,
                           isp_stream_t stream)
{
    isp_status_t s = check_geom(w, h, pitch, out_pitch, 3, 3, border_mode);
    if (s != ISP_OK) return s;
    if (!dx || !dy || !out) return fail(ISP_EINVAL, "null pointer");
    // exact only inside the range of 3x3 Sobel derivatives of u8 images (isp.h): the
    // f32 window sums / f64 response of OpHarris are exact for |v| <= 1020
    if (const_val < -1020 || const_val > 1020)
        return fail(ISP_EINVAL, "harris constant %d outside the Sobel range [-1020,1020]", const_val);
    const size_t ob = img_bytes(w, h, out_pitch, 1);
    if (ranges_overlap(dx, img_bytes(w, h, pitch, 2), out, ob) || ranges_overlap(dy, img_bytes(w, h, pitch, 2), out, ob))
        return fail(ISP_EALIAS, "input and output overlap");
    isp_status_t ts;
    // ISP_TMA / AUTO: the band kernel (band_u8.cu) when eligible, else the tile kernel
    if (tile_variant(3, F_HARRIS, border_mode, w, h, 3, 3, variant,
                     ispi_band_harris_ok(dx, dy, w, h, pitch, out, out_pitch),
                     [&](int *b) { return ispi_harris_band(dx, dy, w, h, pitch, border_mode, const_val, thr, out,
                                                           out_pitch, (cudaStream_t)stream, b); },
                     ts, "isp_harris_u8(band)"))
        return ts;
    if (tile_variant(1, F_HARRIS, border_mode, w, h, 3, 3, variant, ispi_tile_ok(dx, dy, 2, w, h, pitch, out, out_pitch),
                     [&](int *b) { return ispi_harris_tile(dx, dy, w, h, pitch, border_mode, const_val, thr, out,
                                                           out_pitch, (cudaStream_t)stream, b); },
                     ts, "isp_harris_u8(tile)"))
        return ts;
    Desc d = base_desc(w, h, pitch, out_pitch, border_mode, stream);
    d.in0 = dx;
    d.in1 = dy;
    d.out0 = out;
    d.cval_i = const_val;
    d.thr = thr;
    d.mw = d.mh = 3;
    d.g.vec_in = aligned(dx, 2LL * pitch, 8) && aligned(dy, 2LL * pitch, 8);
    d.g.vec_out = aligned(out, out_pitch, 4);
    return resolve_and_launch(d, F_HARRIS, w, h, 3, 3, 1, 1, false, variant, kfn_harris, run_harris,
                              "isp_harris_u8", nullptr,
                              aligned(dx, 2LL * pitch, 16) && aligned(dy, 2LL * pitch, 16), 2, 2);
}

isp_status_t isp_bilateral_f32(const float *img, int w, int h, int pitch, int win, float sigma_d, float sigma_r,
                               int border_mode, float const_val, float *out, int out_pitch, isp_variant_t variant,
                               isp_stream_t stream)
{
    isp_status_t s = check_geom(w, h, pitch, out_pitch, win, win, border_mode);
    if (s != ISP_OK) return s;
    if (!img || !out) return fail(ISP_EINVAL, "null pointer");
    if (!(sigma_d > 0) || !(sigma_r > 0)) return fail(ISP_EINVAL, "sigma must be > 0");
    if (ranges_overlap(img, img_bytes(w, h, pitch, 4), out, img_bytes(w, h, out_pitch, 4)))
        return fail(ISP_EALIAS, "input and output overlap");
    Desc d = base_desc(w, h, pitch, out_pitch, border_mode, stream);
    d.in0 = img;
    d.out0 = out;
    d.cval_f = const_val;
    d.mw = d.mh = win;
    const double LOG2E = 1.4426950408889634;
    d.kr = (float)(-LOG2E / (2.0 * (double)sigma_r * sigma_r));
    std::vector<float> ls((size_t)win * win);
    const int hw = win / 2;
    for (int j = 0; j < win; ++j)
        for (int i = 0; i < win; ++i) {
            const double r2 = (double)(i - hw) * (i - hw) + (double)(j - hw) * (j - hw);
            ls[j * win + i] = (float)(-r2 / (2.0 * (double)sigma_d * sigma_d) * LOG2E);
        }
    d.ls = ls.data();
    d.ax = d.ay = hw;
    d.g.vec_in = 0;
    d.g.vec_out = aligned(out, (long long)out_pitch * 4, 16);
    return resolve_and_launch(d, F_BILATERAL, w, h, win, win, hw, hw, true, variant, kfn_bilateral, run_bilateral,
                              "isp_bilateral_f32");
}

isp_status_t isp_atrous_f32(const float *img, int w, int h, int pitch, int dilation, int border_mode,
                            float const_val, int tonemap, float *out, int out_pitch, isp_variant_t variant,
                            isp_stream_t stream)
{
    if (!(dilation == 1 || dilation == 2 || dilation == 4 || dilation == 8))
        return fail(ISP_EUNSUPPORTED, "dilation %d (built: 1, 2, 4, 8)", dilation);
    isp_status_t s = check_geom(w, h, pitch, out_pitch, 2 * dilation + 1, 2 * dilation + 1, border_mode);
    if (s != ISP_OK) return s;
    if (!img || !out) return fail(ISP_EINVAL, "null pointer");
    if (ranges_overlap(img, img_bytes(w, h, pitch, 4), out, img_bytes(w, h, out_pitch, 4)))
        return fail(ISP_EALIAS, "input and output overlap");
    Desc d = base_desc(w, h, pitch, out_pitch, border_mode, stream);
    d.in0 = img;
    d.out0 = out;
    d.cval_f = const_val;
    d.mw = d.mh = 2 * dilation + 1;
    d.dilation = dilation;
    d.tonemap = tonemap != 0;
    d.g.vec_in = aligned(img, (long long)pitch * 4, 16);
    d.g.vec_out = aligned(out, (long long)out_pitch * 4, 16);
    return resolve_and_launch(d, F_ATROUS, w, h, 3, 3, dilation, dilation, false, variant, kfn_atrous, run_atrous,
                              "isp_atrous_f32");
}

isp_status_t isp_night_f32(const float *img, int w, int h, int pitch, int border_mode, float const_val,
                           float *tmp0, float *tmp1, float *out, int out_pitch, isp_variant_t variant,
                           isp_stream_t stream)
{
    if (!tmp0 || !tmp1) return fail(ISP_EINVAL, "null scratch");
    isp_status_t s;
    if ((s = isp_atrous_f32(img, w, h, pitch, 1, border_mode, const_val, 0, tmp0, out_pitch, variant, stream))) return s;
    if ((s = isp_atrous_f32(tmp0, w, h, out_pitch, 2, border_mode, const_val, 0, tmp1, out_pitch, variant, stream))) return s;
    if ((s = isp_atrous_f32(tmp1, w, h, out_pitch, 4, border_mode, const_val, 0, tmp0, out_pitch, variant, stream))) return s;
    return isp_atrous_f32(tmp0, w, h, out_pitch, 8, border_mode, const_val, 1, out, out_pitch, variant, stream);
}

isp_status_t isp_mask_reach(const void *mask, int dtype, int mw, int mh, int reach[4])
{
    if (!mask || !reach || mw < 1 || mh < 1 || mw > 31 || mh > 31 || (mw % 2) == 0 || (mh % 2) == 0)
        return fail(ISP_EINVAL, "isp_mask_reach args");
    Crop c;
    if (dtype == ISP_F32) {
        std::vector<float> t;
        c = crop_mask((const float *)mask, mw, mh, t);
    } else if (dtype == ISP_I32) {
        std::vector<int32_t> t;
        c = crop_mask((const int32_t *)mask, mw, mh, t);
    } else {
        return fail(ISP_EINVAL, "dtype %d (ISP_F32 or ISP_I32)", dtype);
    }
    std::memcpy(reach, c.reach, sizeof(c.reach));
    return ISP_OK;
}

isp_status_t isp_plan_reach(int w, int h, const int reach[4], int tile_w, int tile_h, int warp_w, isp_plan_info *out)
{
    if (!reach || !out || w < 1 || h < 1 || tile_w < 1 || tile_h < 1) return fail(ISP_EINVAL, "isp_plan_reach args");
    for (int k = 0; k < 4; ++k)
        if (reach[k] < 0 || reach[k] > 30) return fail(ISP_EINVAL, "reach[%d] = %d", k, reach[k]);
    Plan p = make_plan(w, h, reach[0], reach[2], 1, tile_w, tile_h, warp_w > 0 ? warp_w : tile_w, nullptr, 0,
                       reach[1], reach[3]);
    isp_plan_info info{};
    info.bh_l = p.bh_l; info.bh_r = p.bh_r; info.bh_t = p.bh_t; info.bh_b = p.bh_b;
    info.nx = p.nx; info.ny = p.ny; info.w_l = p.w_l; info.w_r = p.w_r;
    info.degenerate = p.degenerate;
    info.tile_w = p.tile_w; info.tile_h = p.ty; info.warp_w = p.warp_w;
    n_block(p, info.n_block);
    info.choice = p.degenerate ? ISP_NAIVE : ISP_BLOCK;
    *out = info;
    return ISP_OK;
}

isp_status_t isp_model_defaults(int filter_id, int border_mode, int mw, int mh, isp_model_params *out)
{
    if (!out) return fail(ISP_EINVAL, "null output");
    (void)mw;
    (void)mh;
    defaults(filter_id, border_mode, *out);
    return ISP_OK;
}

isp_status_t isp_plan(int w, int h, int mw, int mh, int tile_w, int tile_h, int warp_w, int border_mode,
                      int filter_id, const isp_model_params *params, isp_plan_info *out)
{
    isp_status_t s = check_geom(w, h, w, w, mw, mh, border_mode);
    if (s != ISP_OK) return s;
    if (!out) return fail(ISP_EINVAL, "null output");
    const bool direct = (filter_id == F_BILATERAL) || !((mw == mh) && (mw == 3 || mw == 5 || mw == 7));
    int hx = mw / 2, hy = mh / 2;
    Plan p = make_plan(w, h, hx, hy, family_px(filter_id, direct), tile_w, tile_h, warp_w);
    isp_plan_info info{};
    info.bh_l = p.bh_l; info.bh_r = p.bh_r; info.bh_t = p.bh_t; info.bh_b = p.bh_b;
    info.nx = p.nx; info.ny = p.ny; info.w_l = p.w_l; info.w_r = p.w_r;
    info.degenerate = p.degenerate;
    info.tile_w = p.tile_w; info.tile_h = p.ty; info.warp_w = p.warp_w;
    n_block(p, info.n_block);
    isp_model_params mp;
    if (params) mp = *params;
    else defaults(filter_id, border_mode, mp);
    info.o_naive = mp.o_naive > 0 ? mp.o_naive : 1.0;
    info.o_isp = mp.o_isp > 0 ? mp.o_isp : 1.0;
    model(p, w, h, mw, mh, mp, info);
    info.choice = p.degenerate ? ISP_NAIVE : (info.g > 1.0 ? (p.wx > 1 ? ISP_WARP : ISP_BLOCK) : ISP_NAIVE);
    *out = info;
    return ISP_OK;
}

}  // extern "C"
