// shard.cu -- multi-GPU row strips with an NCCL halo exchange (the
// paper is single-GPU).  One process per GPU; torch.distributed only
// bootstraps (broadcast of the ncclUniqueId).
//
// Schedule (isp_shard_schedule, pure host, unit-tested on CPU):
//   rank r owns rows [y0, y0 + strip_h), y0 = r * ceil(H/P);
//   phase 1 "down": send own bottom hy rows to next, receive the top halo from prev;
//   phase 2 "up":   send own top hy rows to prev, receive the bottom halo from next;
//   (prev/next wrap around the ring for Repeat, so no strip has a y border then;
//   per-pair NCCL ordering matches the two phases, also for P = 2);
//   launch 0 (no halo needed): the rows not within hy of a halo edge -- overlaps the
//   exchange; launches 1/2 (after the halo event): the hy rows at each halo edge.
// Only rank 0 owns the image's T border and rank P-1 its B border (Clamp, Mirror,
// Constant); interior ranks run only L / Body / R regions.
#include <cuda.h>
#include <cuda_runtime.h>
#include <nccl.h>

#include <algorithm>
#include <cstring>
#include <vector>

#include "internal.h"

struct isp_shard_ctx {
    ncclComm_t comm;
    int rank, nranks, device;
    cudaEvent_t ev_ready, ev_halo;
};

namespace {

isp_status_t nccl_status(ncclResult_t r, const char *what)
{
    if (r == ncclSuccess) return ISP_OK;
    return ispi_fail(ISP_ENCCL, "%s: %s", what, ncclGetErrorString(r));
}


// The halo exchange of one rank: the schedule's NCCL send/recv calls (bytes of `esz`-byte
// elements, rows of `pitch` elements) in one group on `comm`.
isp_status_t post_exchange(isp_shard_ctx *ctx, const isp_shard_sched &sc, void *strip, size_t esz, int pitch,
                           cudaStream_t comm)
{
    isp_status_t s;
    if ((s = nccl_status(ncclGroupStart(), "ncclGroupStart")) != ISP_OK) return s;
    for (int k = 0; k < sc.n_ops; ++k) {
        const isp_shard_op &op = sc.ops[k];
        char *buf = (char *)strip + (size_t)op.row * pitch * esz;
        const size_t cnt = (size_t)op.nrows * pitch * esz;
        ncclResult_t r = op.kind == 0 ? ncclSend(buf, cnt, ncclUint8, op.peer, ctx->comm, comm)
                                      : ncclRecv(buf, cnt, ncclUint8, op.peer, ctx->comm, comm);
        if (r != ncclSuccess) {
            ncclGroupEnd();
            return nccl_status(r, op.kind == 0 ? "ncclSend" : "ncclRecv");
        }
    }
    return nccl_status(ncclGroupEnd(), "ncclGroupEnd");
}

// ctx == nullptr: local mode (no exchange; the caller filled the halo rows).
template <class T, class F>
isp_status_t shard_run(isp_shard_ctx *ctx, int rank, int nranks, T *strip, int w, int H, int pitch, int halo,
                       int hy, int mode, T *out, int out_pitch, cudaStream_t stream, cudaStream_t comm,
                       F &&filter_rows)
{
    (void)w;
    isp_shard_sched sc;
    isp_status_t s = isp_shard_schedule(H, rank, nranks, halo, hy, mode, &sc);
    if (s != ISP_OK) return s;
    if (!ctx) sc.n_ops = 0;
    if (ctx && cudaSetDevice(ctx->device) != cudaSuccess) return ispi_fail(ISP_ECUDA, "cudaSetDevice");
    if (sc.n_ops > 0) {
        if (cudaEventRecord(ctx->ev_ready, stream) != cudaSuccess ||
            cudaStreamWaitEvent(comm, ctx->ev_ready, 0) != cudaSuccess)
            return ispi_fail(ISP_ECUDA, "event record/wait");
        if ((s = post_exchange(ctx, sc, strip, sizeof(T), pitch, comm)) != ISP_OK) return s;
        if (cudaEventRecord(ctx->ev_halo, comm) != cudaSuccess) return ispi_fail(ISP_ECUDA, "event record");
    }
    // global-row addressing: buffer row k holds global row y0 - halo + k
    const T *in_base = strip - ((ptrdiff_t)sc.y0 - halo) * pitch;
    bool waited = false;
    for (int k = 0; k < sc.n_launch; ++k) {
        const isp_shard_launch &L = sc.launch[k];
        if (L.nrows <= 0) continue;
        if (L.after_halo && !waited && sc.n_ops > 0) {
            if (cudaStreamWaitEvent(stream, ctx->ev_halo, 0) != cudaSuccess)
                return ispi_fail(ISP_ECUDA, "cudaStreamWaitEvent");
            waited = true;
        }
        RowRange rr{L.oy0, L.nrows, L.ylim, L.t_real, L.b_real};
        T *o = out + ((ptrdiff_t)L.oy0 - sc.y0) * out_pitch;
        if ((s = filter_rows(in_base, o, rr)) != ISP_OK) return s;
    }
    if (sc.n_ops > 0 && !waited && cudaStreamWaitEvent(stream, ctx->ev_halo, 0) != cudaSuccess)
        return ispi_fail(ISP_ECUDA, "cudaStreamWaitEvent");
    return ISP_OK;
}

}  // namespace

extern "C" {

isp_status_t isp_shard_rows(int H, int rank, int nranks, int *y0, int *strip_h)
{
    if (H < 1 || nranks < 1 || rank < 0 || rank >= nranks || !y0 || !strip_h)
        return ispi_fail(ISP_EINVAL, "isp_shard_rows(H=%d, rank=%d, nranks=%d)", H, rank, nranks);
    const long long per = ((long long)H + nranks - 1) / nranks;
    const long long a = std::min<long long>(H, per * rank), b = std::min<long long>(H, per * (rank + 1));
    *y0 = (int)a;
    *strip_h = (int)(b - a);
    return ISP_OK;
}

isp_status_t isp_shard_schedule(int H, int rank, int nranks, int halo, int hy, int border_mode,
                                isp_shard_sched *out)
{
    if (!out) return ispi_fail(ISP_EINVAL, "null output");
    if (border_mode < 0 || border_mode > 3 || hy < 0 || halo < hy)
        return ispi_fail(ISP_EINVAL, "schedule: mode %d, hy %d, halo %d", border_mode, hy, halo);
    isp_shard_sched sc;
    std::memset(&sc, 0, sizeof(sc));
    isp_status_t s = isp_shard_rows(H, rank, nranks, &sc.y0, &sc.strip_h);
    if (s != ISP_OK) return s;
    // every strip must hold its own two halo bands (and feed its neighbours)
    for (int r = 0; r < nranks; ++r) {
        int a, b;
        isp_shard_rows(H, r, nranks, &a, &b);
        if (nranks > 1 && b < std::max(2 * hy, 1))
            return ispi_fail(ISP_EINVAL, "strip of rank %d has %d rows < 2*hy = %d", r, b, 2 * hy);
    }
    const bool ring = border_mode == ISP_REPEAT && nranks > 1;
    const int prev = rank > 0 ? rank - 1 : (ring ? nranks - 1 : -1);
    const int next = rank < nranks - 1 ? rank + 1 : (ring ? 0 : -1);
    sc.prev = prev;
    sc.next = next;
    const int sh = sc.strip_h;
    if (hy > 0) {
        // phase 1 (down), phase 2 (up) -- see file header for the per-pair ordering
        if (next >= 0) sc.ops[sc.n_ops++] = isp_shard_op{0, next, halo + sh - hy, hy};
        if (prev >= 0) sc.ops[sc.n_ops++] = isp_shard_op{1, prev, halo - hy, hy};
        if (prev >= 0) sc.ops[sc.n_ops++] = isp_shard_op{0, prev, halo, hy};
        if (next >= 0) sc.ops[sc.n_ops++] = isp_shard_op{1, next, halo + sh, hy};
    }
    const int need_top = prev >= 0 ? hy : 0, need_bot = next >= 0 ? hy : 0;
    const int t_real = prev < 0, b_real = next < 0;
    const int y0 = sc.y0;
    // launch 0: rows that need no halo; reads only own rows (ylim = strip end)
    sc.launch[sc.n_launch++] = isp_shard_launch{y0 + need_top, sh - need_top - need_bot, y0 + sh, t_real, b_real, 0};
    if (need_top)
        sc.launch[sc.n_launch++] = isp_shard_launch{y0, need_top, y0 + sh, 0, 0, 1};
    if (need_bot)
        sc.launch[sc.n_launch++] = isp_shard_launch{y0 + sh - need_bot, need_bot, y0 + sh + need_bot, 0, 0, 1};
    *out = sc;
    return ISP_OK;
}

isp_status_t isp_shard_unique_id(unsigned char id[128])
{
    if (!id) return ispi_fail(ISP_EINVAL, "null id");
    ncclUniqueId uid;
    isp_status_t s = nccl_status(ncclGetUniqueId(&uid), "ncclGetUniqueId");
    if (s != ISP_OK) return s;
    static_assert(sizeof(uid.internal) == 128, "ncclUniqueId size");
    std::memcpy(id, uid.internal, 128);
    return ISP_OK;
}

isp_status_t isp_shard_init(isp_shard_ctx **ctx, const unsigned char id[128], int rank, int nranks, int device)
{
    if (!ctx || !id || nranks < 1 || rank < 0 || rank >= nranks) return ispi_fail(ISP_EINVAL, "isp_shard_init args");
    if (cudaSetDevice(device) != cudaSuccess) return ispi_fail(ISP_ECUDA, "cudaSetDevice(%d)", device);
    isp_shard_ctx *c = new isp_shard_ctx{};
    c->rank = rank;
    c->nranks = nranks;
    c->device = device;
    ncclUniqueId uid;
    std::memcpy(uid.internal, id, 128);
    isp_status_t s = nccl_status(ncclCommInitRank(&c->comm, nranks, uid, rank), "ncclCommInitRank");
    if (s != ISP_OK) {
        delete c;
        return s;
    }
    if (cudaEventCreateWithFlags(&c->ev_ready, cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreateWithFlags(&c->ev_halo, cudaEventDisableTiming) != cudaSuccess) {
        ncclCommDestroy(c->comm);
        delete c;
        return ispi_fail(ISP_ECUDA, "cudaEventCreate");
    }
    *ctx = c;
    return ISP_OK;
}

isp_status_t isp_shard_filter_local_f32(float *strip, int w, int H, int pitch, int halo, int rank, int nranks,
                                        const float *mask, int mw, int mh, int border_mode, float const_val,
                                        float *out, int out_pitch, isp_variant_t variant, isp_stream_t stream)
{
    if (!strip || !out || !mask) return ispi_fail(ISP_EINVAL, "null pointer");
    auto f = [&](const float *in_base, float *o, const RowRange &rr) {
        return ispi_filter_f32(in_base, w, H, pitch, mask, mw, mh, border_mode, const_val, o, out_pitch, variant,
                               stream, &rr);
    };
    return shard_run<float>(nullptr, rank, nranks, strip, w, H, pitch, halo, mh / 2, border_mode, out, out_pitch,
                            (cudaStream_t)stream, (cudaStream_t)stream, f);
}

isp_status_t isp_shard_filter_local_u8(uint8_t *strip, int w, int H, int pitch, int halo, int rank, int nranks,
                                       const int32_t *mask, int mw, int mh, int32_t divisor, int border_mode,
                                       int const_val, uint8_t *out, int out_pitch, isp_variant_t variant,
                                       isp_stream_t stream)
{
    if (!strip || !out || !mask) return ispi_fail(ISP_EINVAL, "null pointer");
    auto f = [&](const uint8_t *in_base, uint8_t *o, const RowRange &rr) {
        return ispi_filter_u8(in_base, w, H, pitch, mask, mw, mh, divisor, border_mode, const_val, o, out_pitch,
                              variant, stream, &rr);
    };
    return shard_run<uint8_t>(nullptr, rank, nranks, strip, w, H, pitch, halo, mh / 2, border_mode, out, out_pitch,
                              (cudaStream_t)stream, (cudaStream_t)stream, f);
}

isp_status_t isp_shard_exchange(isp_shard_ctx *ctx, void *strip, int elem_size, int H, int pitch, int halo, int hy,
                                int border_mode, isp_stream_t comm_stream)
{
    if (!ctx || !strip || elem_size < 1 || pitch < 1) return ispi_fail(ISP_EINVAL, "isp_shard_exchange args");
    isp_shard_sched sc;
    isp_status_t s = isp_shard_schedule(H, ctx->rank, ctx->nranks, halo, hy, border_mode, &sc);
    if (s != ISP_OK) return s;
    if (cudaSetDevice(ctx->device) != cudaSuccess) return ispi_fail(ISP_ECUDA, "cudaSetDevice");
    return sc.n_ops > 0 ? post_exchange(ctx, sc, strip, (size_t)elem_size, pitch, (cudaStream_t)comm_stream) : ISP_OK;
}

}  // extern "C"

// ---------------------------------------------------------------------------------
// Peer-direct strips: no halo rows, no exchange.  Each rank's strip
// holds only its own rows; the launch reads the hy rows above / below straight from the
// neighbours' strips (peer memory over NVLink: CUDA IPC across processes, or any pointer
// the device can dereference), so one launch covers the whole strip and nothing waits for
// communication.  The strip-edge block rows are T / B regions that select the neighbour
// buffer per row (row_base in isp_core.cuh); Body rows never leave the strip.
// ---------------------------------------------------------------------------------
namespace {

template <class T>
isp_status_t peer_rowrange(const T *own, const T *prev, const T *next, int H, int pitch, int rank, int nranks,
                           int hy, int mode, RowRange &rr, const T *&base)
{
    int y0, sh;
    isp_status_t s = isp_shard_rows(H, rank, nranks, &y0, &sh);
    if (s != ISP_OK) return s;
    const bool ring = mode == ISP_REPEAT && nranks > 1;
    const int pr = rank > 0 ? rank - 1 : (ring ? nranks - 1 : -1);
    const int nx = rank < nranks - 1 ? rank + 1 : (ring ? 0 : -1);
    for (int r : {pr, nx}) {
        if (r < 0) continue;
        int a, b;
        isp_shard_rows(H, r, nranks, &a, &b);
        if (b < hy) return ispi_fail(ISP_EINVAL, "peer strip of rank %d has %d rows < hy = %d", r, b, hy);
    }
    if ((pr >= 0 && !prev) || (nx >= 0 && !next)) return ispi_fail(ISP_EINVAL, "missing neighbour strip pointer");
    rr = RowRange{y0, sh, y0 + sh + hy, pr < 0, nx < 0};
    rr.peer = 1;
    rr.own_y0 = y0;
    rr.own_y1 = y0 + sh;
    base = own - (ptrdiff_t)y0 * pitch;
    if (pr >= 0) {   // rows y < y0 of rank pr (rank 0 in a ring: global rows y + H)
        int py0, psh;
        isp_shard_rows(H, pr, nranks, &py0, &psh);
        rr.peer_lo = prev - ((ptrdiff_t)py0 - (rank == 0 ? H : 0)) * pitch;
    }
    if (nx >= 0) {   // rows y >= y0 + sh of rank nx (last rank in a ring: global rows y - H)
        int ny0, nsh;
        isp_shard_rows(H, nx, nranks, &ny0, &nsh);
        rr.peer_hi = next - ((ptrdiff_t)ny0 + (rank == nranks - 1 ? H : 0)) * pitch;
    }
    return ISP_OK;
}

}  // namespace

extern "C" {

isp_status_t isp_shard_filter_peer_local_f32(const float *own, const float *prev, const float *next, int w, int H,
                                             int pitch, int rank, int nranks, const float *mask, int mw, int mh,
                                             int border_mode, float const_val, float *out, int out_pitch,
                                             isp_variant_t variant, isp_stream_t stream)
{
    if (!own || !out || !mask) return ispi_fail(ISP_EINVAL, "null pointer");
    if (border_mode < 0 || border_mode > 3) return ispi_fail(ISP_EINVAL, "border mode %d", border_mode);
    RowRange rr{};
    const float *base = nullptr;
    isp_status_t s = peer_rowrange(own, prev, next, H, pitch, rank, nranks, mh / 2, border_mode, rr, base);
    if (s != ISP_OK) return s;
    return ispi_filter_f32(base, w, H, pitch, mask, mw, mh, border_mode, const_val, out, out_pitch, variant, stream,
                           &rr);
}

isp_status_t isp_shard_filter_peer_local_u8(const uint8_t *own, const uint8_t *prev, const uint8_t *next, int w,
                                            int H, int pitch, int rank, int nranks, const int32_t *mask, int mw,
                                            int mh, int32_t divisor, int border_mode, int const_val, uint8_t *out,
                                            int out_pitch, isp_variant_t variant, isp_stream_t stream)
{
    if (!own || !out || !mask) return ispi_fail(ISP_EINVAL, "null pointer");
    if (border_mode < 0 || border_mode > 3) return ispi_fail(ISP_EINVAL, "border mode %d", border_mode);
    RowRange rr{};
    const uint8_t *base = nullptr;
    isp_status_t s = peer_rowrange(own, prev, next, H, pitch, rank, nranks, mh / 2, border_mode, rr, base);
    if (s != ISP_OK) return s;
    return ispi_filter_u8(base, w, H, pitch, mask, mw, mh, divisor, border_mode, const_val, out, out_pitch, variant,
                          stream, &rr);
}

}  // extern "C"

struct isp_shard_peer {
    int rank, nranks, device;
    void *own;
    void *prev, *next;        // neighbour strips (opened IPC mappings), or null
    void *prev_base, *next_base;
};

namespace {
struct PeerInfo {                    // 72 bytes: IPC handle of the allocation + offset
    cudaIpcMemHandle_t h;
    unsigned long long off;
};
static_assert(sizeof(PeerInfo) == 72, "peer handle layout");
}  // namespace

extern "C" {

isp_status_t isp_shard_peer_handle(void *strip, unsigned char out[72])
{
    if (!strip || !out) return ispi_fail(ISP_EINVAL, "isp_shard_peer_handle args");
    // allocation base of the strip (IPC handles name allocations; torch's caching
    // allocator hands out sub-ranges): cuMemGetAddressRange through the runtime's driver
    // entry point, so libisp.so does not link libcuda (CPU boxes load it without a driver)
    using AddrRangeFn = CUresult (*)(CUdeviceptr *, size_t *, CUdeviceptr);
    void *fnp = nullptr;
    cudaDriverEntryPointQueryResult q{};
    if (cudaGetDriverEntryPoint("cuMemGetAddressRange", &fnp, cudaEnableDefault, &q) != cudaSuccess || !fnp)
        return ispi_fail(ISP_ECUDA, "cuMemGetAddressRange entry point unavailable");
    CUdeviceptr base = 0;
    size_t size = 0;
    if (((AddrRangeFn)fnp)(&base, &size, (CUdeviceptr)strip) != CUDA_SUCCESS)
        return ispi_fail(ISP_ECUDA, "cuMemGetAddressRange of the strip failed");
    PeerInfo mine{};
    cudaError_t e = cudaIpcGetMemHandle(&mine.h, (void *)base);
    if (e != cudaSuccess) return ispi_fail(ISP_ECUDA, "cudaIpcGetMemHandle: %s", cudaGetErrorString(e));
    mine.off = (unsigned long long)((CUdeviceptr)strip - base);
    std::memcpy(out, &mine, sizeof(mine));
    return ISP_OK;
}

isp_status_t isp_shard_peer_attach(int rank, int nranks, int device, void *strip, const unsigned char *handles,
                                   int ring, isp_shard_peer **out)
{
    if (!strip || !handles || !out || nranks < 1 || rank < 0 || rank >= nranks)
        return ispi_fail(ISP_EINVAL, "isp_shard_peer_attach args");
    if (cudaSetDevice(device) != cudaSuccess) return ispi_fail(ISP_ECUDA, "cudaSetDevice(%d)", device);
    std::vector<PeerInfo> all(nranks);
    std::memcpy(all.data(), handles, sizeof(PeerInfo) * nranks);
    isp_shard_peer *pp = new isp_shard_peer{};
    pp->rank = rank;
    pp->nranks = nranks;
    pp->device = device;
    pp->own = strip;
    const int P = nranks, r = rank;
    const int pr = r > 0 ? r - 1 : ((ring && P > 1) ? P - 1 : -1);
    const int nx = r < P - 1 ? r + 1 : ((ring && P > 1) ? 0 : -1);
    auto open = [&](int q, void *&basep, void *&ptr) -> isp_status_t {
        if (q < 0 || q == r) return ISP_OK;
        cudaError_t ee = cudaIpcOpenMemHandle(&basep, all[q].h, cudaIpcMemLazyEnablePeerAccess);
        if (ee != cudaSuccess) {
            cudaGetLastError();
            return ispi_fail(ISP_ECUDA, "cudaIpcOpenMemHandle(rank %d): %s", q, cudaGetErrorString(ee));
        }
        ptr = (char *)basep + all[q].off;
        return ISP_OK;
    };
    isp_status_t s = open(pr, pp->prev_base, pp->prev);
    if (s == ISP_OK) {
        if (nx == pr && nx >= 0) {   // P = 2 ring: one mapping serves both sides
            pp->next = pp->prev;
        } else {
            s = open(nx, pp->next_base, pp->next);
        }
    }
    if (s != ISP_OK) {
        isp_shard_peer_close(pp);
        return s;
    }
    *out = pp;
    return ISP_OK;
}

isp_status_t isp_shard_peer_open(isp_shard_ctx *ctx, void *strip, int ring, isp_shard_peer **out)
{
    if (!ctx || !strip || !out) return ispi_fail(ISP_EINVAL, "isp_shard_peer_open args");
    if (cudaSetDevice(ctx->device) != cudaSuccess) return ispi_fail(ISP_ECUDA, "cudaSetDevice");
    PeerInfo mine{};
    isp_status_t s = isp_shard_peer_handle(strip, reinterpret_cast<unsigned char *>(&mine));
    if (s != ISP_OK) return s;
    const int P = ctx->nranks;
    PeerInfo *dsend = nullptr, *drecv = nullptr;
    std::vector<PeerInfo> all(P);
    cudaStream_t st;
    if (cudaMalloc(&dsend, sizeof(PeerInfo)) != cudaSuccess || cudaMalloc(&drecv, sizeof(PeerInfo) * P) != cudaSuccess ||
        cudaStreamCreate(&st) != cudaSuccess)
        return ispi_fail(ISP_ECUDA, "peer handle exchange buffers");
    cudaMemcpy(dsend, &mine, sizeof(PeerInfo), cudaMemcpyHostToDevice);
    s = nccl_status(ncclAllGather(dsend, drecv, sizeof(PeerInfo), ncclUint8, ctx->comm, st), "ncclAllGather(ipc handles)");
    if (s == ISP_OK && cudaStreamSynchronize(st) != cudaSuccess) s = ispi_fail(ISP_ECUDA, "handle exchange");
    if (s == ISP_OK) cudaMemcpy(all.data(), drecv, sizeof(PeerInfo) * P, cudaMemcpyDeviceToHost);
    cudaFree(dsend);
    cudaFree(drecv);
    cudaStreamDestroy(st);
    if (s != ISP_OK) return s;
    return isp_shard_peer_attach(ctx->rank, P, ctx->device, strip, reinterpret_cast<const unsigned char *>(all.data()),
                                 ring, out);
}

isp_status_t isp_shard_peer_filter_f32(isp_shard_peer *pp, int w, int H, int pitch, const float *mask, int mw, int mh,
                                       int border_mode, float const_val, float *out, int out_pitch,
                                       isp_variant_t variant, isp_stream_t stream)
{
    if (!pp) return ispi_fail(ISP_EINVAL, "null peer context");
    if (cudaSetDevice(pp->device) != cudaSuccess) return ispi_fail(ISP_ECUDA, "cudaSetDevice");
    return isp_shard_filter_peer_local_f32((const float *)pp->own, (const float *)pp->prev, (const float *)pp->next, w,
                                           H, pitch, pp->rank, pp->nranks, mask, mw, mh, border_mode, const_val, out,
                                           out_pitch, variant, stream);
}

isp_status_t isp_shard_peer_close(isp_shard_peer *pp)
{
    if (!pp) return ISP_OK;
    if (pp->prev_base) cudaIpcCloseMemHandle(pp->prev_base);
    if (pp->next_base && pp->next_base != pp->prev_base) cudaIpcCloseMemHandle(pp->next_base);
    delete pp;
    return ISP_OK;
}

isp_status_t isp_shard_destroy(isp_shard_ctx *ctx)
{
    if (!ctx) return ISP_OK;
    cudaEventDestroy(ctx->ev_ready);
    cudaEventDestroy(ctx->ev_halo);
    ncclResult_t r = ncclCommDestroy(ctx->comm);
    delete ctx;
    return nccl_status(r, "ncclCommDestroy");
}

isp_status_t isp_shard_filter_f32(isp_shard_ctx *ctx, float *strip, int w, int H, int pitch, int halo,
                                  const float *mask, int mw, int mh, int border_mode, float const_val, float *out,
                                  int out_pitch, isp_variant_t variant, isp_stream_t stream, isp_stream_t comm_stream)
{
    if (!ctx || !strip || !out || !mask) return ispi_fail(ISP_EINVAL, "null pointer");
    auto f = [&](const float *in_base, float *o, const RowRange &rr) {
        return ispi_filter_f32(in_base, w, H, pitch, mask, mw, mh, border_mode, const_val, o, out_pitch, variant,
                               stream, &rr);
    };
    return shard_run<float>(ctx, ctx->rank, ctx->nranks, strip, w, H, pitch, halo, mh / 2, border_mode, out, out_pitch,
                            (cudaStream_t)stream, (cudaStream_t)comm_stream, f);
}

isp_status_t isp_shard_filter_u8(isp_shard_ctx *ctx, uint8_t *strip, int w, int H, int pitch, int halo,
                                 const int32_t *mask, int mw, int mh, int32_t divisor, int border_mode, int const_val,
                                 uint8_t *out, int out_pitch, isp_variant_t variant, isp_stream_t stream,
                                 isp_stream_t comm_stream)
{
    if (!ctx || !strip || !out || !mask) return ispi_fail(ISP_EINVAL, "null pointer");
    auto f = [&](const uint8_t *in_base, uint8_t *o, const RowRange &rr) {
        return ispi_filter_u8(in_base, w, H, pitch, mask, mw, mh, divisor, border_mode, const_val, o, out_pitch,
                              variant, stream, &rr);
    };
    return shard_run<uint8_t>(ctx, ctx->rank, ctx->nranks, strip, w, H, pitch, halo, mh / 2, border_mode, out,
                              out_pitch, (cudaStream_t)stream, (cudaStream_t)comm_stream, f);
}

}  // extern "C"
