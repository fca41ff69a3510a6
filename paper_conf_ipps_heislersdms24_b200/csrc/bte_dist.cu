// bte_dist.cu -- the multi-rank exchanges (see bte_internal.h): the band
// coupling of the step across ranks (L760-766; reduce-scatter of
// the energy, chunk solves, all-gather of T, or one all-reduce), the halo
// exchange of cell partitions (L728-735, L768-772), the dt
// bound agreement, and the cell-partition ABI.
#include "bte_internal.h"

namespace bte_host {


bte_status allreduce_E(bte_ctx *ctx, double *E) {
    if (!ctx->have_bcomm) return BTE_OK;
    std::string e;
    if (!bte::nccl::allreduce_sum_f64(ctx->bcomm, E ? E : ctx->E, ctx->nc, ctx->stream, &e)) {
        set_err(&ctx->err, "NCCL all-reduce failed: %s", e.c_str());
        return BTE_ENCCL;
    }
    return BTE_OK;
}

// Band-sharded step exchange (SURVEY 8(e) alternative, no replicated solve):
// E (slot sum, padded to world x chunk) -> reduce-scatter -> Newton on this
// rank's chunk of cells -> all-gather of T -> every rank finishes its rows.
bte_status shard_newton_step(bte_ctx *ctx) {
    std::string e;
    ev_mark(ctx, kPhAllreduce, true);
    STATUS_TRY(reduce_slots(ctx));
    if (!bte::nccl::reduce_scatter_sum_f64(ctx->bcomm, ctx->E, ctx->Echunk, ctx->chunk, ctx->stream, &e))
        return set_err(&ctx->err, "NCCL reduce-scatter failed: %s", e.c_str()), BTE_ENCCL;
    ev_mark(ctx, kPhAllreduce, false);
    ev_mark(ctx, kPhNewton, true);
    bte::NewtonParams q = newton_params(ctx, ctx->Echunk, /*step=*/true);
    q.c_lo = ctx->gband * ctx->chunk;
    q.nc = std::max(0, std::min(ctx->chunk, ctx->nc - q.c_lo));
    q.T_out = ctx->Tg;
    q.neg_fail = 1;
    q.spec = 0;  // (a chunk of cells: the finish kernel refreshes every row after the all-gather)
    if (warp_newton(ctx, q.nc)) STATUS_TRY(launch_newton_warp(ctx, q));
    else STATUS_TRY(launch_newton_cells(ctx, q));
    double *mine = ctx->Tg + (size_t)ctx->gband * ctx->chunk;
    if (!bte::nccl::allgather_f64(ctx->bcomm, mine, ctx->Tg, ctx->chunk, ctx->stream, &e))
        return set_err(&ctx->err, "NCCL all-gather failed: %s", e.c_str()), BTE_ENCCL;
    STATUS_TRY(newton_finish(ctx));
    ev_mark(ctx, kPhNewton, false);
    if (ctx->td && !ctx->rate_now) ctx->rsel = 1 - ctx->rsel;
    CUDA_TRY(ctx, cudaGetLastError());
    return BTE_OK;
}

// ------------------------------------------------------------- halo (N3)
// Pack / unpack one segment for every local band-row (current slabs).
bte::HaloParams halo_params(const bte_ctx *ctx) {
    bte::HaloParams hp{};
    for (int k = 0; k < ctx->nb_loc; ++k) hp.row[k] = ctx->pool_cells + (int64_t)ctx->cur_slot[k] * ctx->slab_elems;
    hp.nb_loc = ctx->nb_loc;
    hp.ps = ctx->ps;
    hp.fail = ctx->d_fail;
    return hp;
}

dim3 halo_grid(const bte_ctx *ctx, int64_t per) {
    return dim3((unsigned)std::max<int64_t>(1, std::min<int64_t>(2048, (per + 255) / 256)), (unsigned)ctx->nb_loc);
}

bte_status halo_pack(bte_ctx *ctx, const HaloSeg &h) {
    if (h.n_send() == 0) return BTE_OK;
    bte::HaloParams hp = halo_params(ctx);
    hp.cells = h.send_cells;
    hp.dirs = h.send_dirs;
    hp.n = h.n_send_cells;
    hp.n_dirs = h.n_send_dirs;
    bte::halo_pack_kernel<<<halo_grid(ctx, h.n_send()), 256, 0, ctx->stream>>>(hp, h.sbuf);
    ctx->st.kernel_launches++;
    CUDA_TRY(ctx, cudaGetLastError());
    return BTE_OK;
}

bte_status halo_unpack(bte_ctx *ctx, const HaloSeg &h) {
    if (h.n_recv() == 0) return BTE_OK;
    bte::HaloParams hp = halo_params(ctx);
    hp.dirs = h.recv_dirs;
    hp.n = h.n_recv_cells;
    hp.n_dirs = h.n_recv_dirs;
    hp.cells = h.recv_cols;
    bte::halo_unpack_kernel<<<halo_grid(ctx, h.n_recv()), 256, 0, ctx->stream>>>(hp, h.rbuf);
    ctx->st.kernel_launches++;
    CUDA_TRY(ctx, cudaGetLastError());
    return BTE_OK;
}

// Cell-partitioned step, before the flux: every segment packed, one NCCL group
// of sends / receives with the neighbour parts of this band group, unpacked
// into the halo columns of the current slabs (I^n, the old level, Eq. 3).
bte_status halo_exchange(bte_ctx *ctx) {
    if (ctx->hsegs.empty()) return BTE_OK;
    if (!ctx->have_comm) return set_err(&ctx->err, "halo exchange needs a communicator"), BTE_ESTATE;
    ev_mark(ctx, kPhHalo, true);
    for (const HaloSeg &h : ctx->hsegs) STATUS_TRY(halo_pack(ctx, h));
    std::vector<bte::nccl::P2P> ops;
    for (const HaloSeg &h : ctx->hsegs)
        ops.push_back({ctx->gband * ctx->n_parts + h.part, h.sbuf, h.n_send() * ctx->nb_loc, h.rbuf,
                       h.n_recv() * ctx->nb_loc});
    std::string e;
    if (!bte::nccl::exchange_f64(ctx->comm, ops.data(), (int)ops.size(), ctx->stream, &e))
        return set_err(&ctx->err, "NCCL halo exchange failed: %s", e.c_str()), BTE_ENCCL;
    for (const HaloSeg &h : ctx->hsegs) STATUS_TRY(halo_unpack(ctx, h));
    ev_mark(ctx, kPhHalo, false);
    return BTE_OK;
}

// With the rate law the bound depends on the hottest temperature the state can
// reach (t_hi); under cell partitioning each rank only sees its own cells, so
// the ranks agree on the max first (every bte_step of such a run is collective
// anyway), and all of them accept or reject the same dt.
bte_status sync_dt_bound(bte_ctx *ctx) {
    if (!(ctx->td && ctx->n_parts > 1 && ctx->have_comm)) return BTE_OK;
    double *d = reinterpret_cast<double *>(ctx->d_smax);
    CUDA_TRY(ctx, cudaMemcpyAsync(d, &ctx->t_hi, sizeof(double), cudaMemcpyHostToDevice, ctx->stream));
    std::string e;
    if (!bte::nccl::allreduce_max_f64(ctx->comm, d, 1, ctx->stream, &e))
        return set_err(&ctx->err, "all-reduce (max) of the hottest temperature failed: %s", e.c_str()), BTE_ENCCL;
    CUDA_TRY(ctx, cudaMemcpyAsync(&ctx->t_hi, d, sizeof(double), cudaMemcpyDeviceToHost, ctx->stream));
    CUDA_TRY(ctx, cudaStreamSynchronize(ctx->stream));
    update_dt_bound(ctx);
    return BTE_OK;
}

}  // namespace bte_host

using namespace bte_host;

extern "C" {


bte_status bte_local_cells(const bte_ctx *ctx, int64_t *n_local, int64_t *ids) {
    if (!ctx || !n_local) return BTE_EINVAL;
    *n_local = ctx->nc;
    if (ids)
        for (int32_t i = 0; i < ctx->nc; ++i) ids[i] = ctx->gid.empty() ? i : ctx->gid[i];
    return BTE_OK;
}

static const HaloSeg *find_seg(const bte_ctx *ctx, int32_t part, bte_status *st) {
    *st = BTE_OK;
    if (part < 0 || part >= ctx->n_parts) {
        set_err(const_cast<std::string *>(&ctx->err), "part %d outside [0, %d)", part, ctx->n_parts);
        *st = BTE_EINVAL;
        return nullptr;
    }
    for (const HaloSeg &h : ctx->hsegs)
        if (h.part == part) return &h;
    return nullptr;  // no shared face: empty segment
}

bte_status bte_halo_size(const bte_ctx *ctx, int32_t part, int64_t *n_send, int64_t *n_recv) {
    if (!ctx || !n_send || !n_recv) return BTE_EINVAL;
    bte_status st;
    const HaloSeg *h = find_seg(ctx, part, &st);
    STATUS_TRY(st);
    *n_send = h ? h->n_send() * ctx->nb_loc : 0;
    *n_recv = h ? h->n_recv() * ctx->nb_loc : 0;
    return BTE_OK;
}

bte_status bte_halo_export(const bte_ctx *cctx, int32_t part, double *buf) {
    if (!cctx || !buf) return BTE_EINVAL;
    bte_ctx *ctx = const_cast<bte_ctx *>(cctx);
    if (ctx->begun) return set_err(&ctx->err, "split step in flight"), BTE_ESTATE;
    bte_status st;
    const HaloSeg *h = find_seg(ctx, part, &st);
    STATUS_TRY(st);
    if (!h || h->n_send() == 0) return BTE_OK;
    CUDA_TRY(ctx, cudaSetDevice(ctx->device));
    STATUS_TRY(halo_pack(ctx, *h));
    CUDA_TRY(ctx, cudaMemcpyAsync(buf, h->sbuf, (size_t)h->n_send() * ctx->nb_loc * sizeof(double),
                                  cudaMemcpyDeviceToHost, ctx->stream));
    CUDA_TRY(ctx, cudaStreamSynchronize(ctx->stream));
    return BTE_OK;
}

bte_status bte_halo_import(bte_ctx *ctx, int32_t part, const double *buf) {
    if (!ctx || !buf) return BTE_EINVAL;
    if (ctx->begun) return set_err(&ctx->err, "split step in flight"), BTE_ESTATE;
    bte_status st;
    const HaloSeg *h = find_seg(ctx, part, &st);
    STATUS_TRY(st);
    if (!h || h->n_recv() == 0) return BTE_OK;
    CUDA_TRY(ctx, cudaSetDevice(ctx->device));
    CUDA_TRY(ctx, cudaMemcpyAsync(h->rbuf, buf, (size_t)h->n_recv() * ctx->nb_loc * sizeof(double),
                                  cudaMemcpyHostToDevice, ctx->stream));
    STATUS_TRY(halo_unpack(ctx, *h));
    CUDA_TRY(ctx, cudaStreamSynchronize(ctx->stream));
    return BTE_OK;
}

}  // extern "C"
