// bte_state.cu -- getters, setters, re-solves and counters (see bte_internal.h).
#include "bte_internal.h"
#include <cfloat>


using namespace bte_host;

extern "C" {


bte_status bte_dt_bound(const bte_ctx *ctx, double *dt_max) {
    if (!ctx || !dt_max) return BTE_EINVAL;
    *dt_max = ctx->dt_bound;
    return BTE_OK;
}

bte_status bte_band_range(const bte_ctx *ctx, int32_t *b_lo, int32_t *b_hi) {
    if (!ctx || !b_lo || !b_hi) return BTE_EINVAL;
    *b_lo = ctx->b_lo;
    *b_hi = ctx->b_hi;
    return BTE_OK;
}

// rows of nc doubles (device rows of `stride` elements, internal order) <-> host (caller order)
static bte_status rows_to_host(const bte_ctx *cctx, const double *dsrc, int64_t stride, int64_t rows, double *host) {
    bte_ctx *ctx = const_cast<bte_ctx *>(cctx);
    if (ctx->identity_order) {  // one strided copy, no gather (and no staging round trip)
        CUDA_TRY(ctx, cudaMemcpy2DAsync(host, ctx->nc * sizeof(double), dsrc, stride * sizeof(double),
                                        ctx->nc * sizeof(double), rows, cudaMemcpyDeviceToHost, ctx->stream));
        CUDA_TRY(ctx, cudaStreamSynchronize(ctx->stream));
        return BTE_OK;
    }
    const int64_t per = std::max<int64_t>(1, ctx->staging_elems / ctx->nc);
    for (int64_t r0 = 0; r0 < rows; r0 += per) {
        const int64_t nr = std::min(per, rows - r0);
        const int64_t n = nr * ctx->nc;
        const int tb = 256;
        const int gb = (int)std::min<int64_t>(8192, (n + tb - 1) / tb);
        bte::gather_rows_kernel<<<gb, tb, 0, ctx->stream>>>(dsrc + r0 * stride, ctx->pos, ctx->nc, stride, nr,
                                                            ctx->staging);
        CUDA_TRY(ctx, cudaGetLastError());
        CUDA_TRY(ctx, cudaMemcpyAsync(host + r0 * ctx->nc, ctx->staging, n * sizeof(double), cudaMemcpyDeviceToHost,
                                      ctx->stream));
        CUDA_TRY(ctx, cudaStreamSynchronize(ctx->stream));
    }
    return BTE_OK;
}

static bte_status rows_from_host(bte_ctx *ctx, const double *host, int64_t stride, int64_t rows, double *ddst) {
    if (ctx->identity_order) {  // one strided copy, no scatter (and no staging round trip)
        CUDA_TRY(ctx, cudaMemcpy2DAsync(ddst, stride * sizeof(double), host, ctx->nc * sizeof(double),
                                        ctx->nc * sizeof(double), rows, cudaMemcpyHostToDevice, ctx->stream));
        CUDA_TRY(ctx, cudaStreamSynchronize(ctx->stream));
        return BTE_OK;
    }
    const int64_t per = std::max<int64_t>(1, ctx->staging_elems / ctx->nc);
    for (int64_t r0 = 0; r0 < rows; r0 += per) {
        const int64_t nr = std::min(per, rows - r0);
        const int64_t n = nr * ctx->nc;
        CUDA_TRY(ctx, cudaMemcpyAsync(ctx->staging, host + r0 * ctx->nc, n * sizeof(double), cudaMemcpyHostToDevice,
                                      ctx->stream));
        const int tb = 256;
        const int gb = (int)std::min<int64_t>(8192, (n + tb - 1) / tb);
        bte::scatter_rows_kernel<<<gb, tb, 0, ctx->stream>>>(ctx->staging, ctx->pos, ctx->nc, stride, nr,
                                                             ddst + r0 * stride);
        CUDA_TRY(ctx, cudaGetLastError());
        CUDA_TRY(ctx, cudaStreamSynchronize(ctx->stream));
    }
    return BTE_OK;
}

bte_status bte_get_temperature(const bte_ctx *ctx, double *T) {
    if (!ctx || !T) return BTE_EINVAL;
    CUDA_TRY(const_cast<bte_ctx *>(ctx), cudaSetDevice(ctx->device));
    return rows_to_host(ctx, ctx->T, ctx->nc, 1, T);
}

bte_status bte_get_energy(const bte_ctx *ctx, double *E) {
    if (!ctx || !E) return BTE_EINVAL;
    CUDA_TRY(const_cast<bte_ctx *>(ctx), cudaSetDevice(ctx->device));
    return rows_to_host(ctx, ctx->E, ctx->nc, 1, E);
}

bte_status bte_set_energy(bte_ctx *ctx, const double *E) {
    if (!ctx || !E) return BTE_EINVAL;
    CUDA_TRY(ctx, cudaSetDevice(ctx->device));
    return rows_from_host(ctx, E, ctx->nc, 1, ctx->E);
}

static bte_status check_rows(const bte_ctx *ctx, int32_t b_lo, int32_t b_hi) {
    if (b_lo < ctx->b_lo || b_hi > ctx->b_hi || b_lo >= b_hi) {
        set_err(const_cast<std::string *>(&ctx->err), "band-rows [%d,%d) outside this rank's [%d,%d)", b_lo, b_hi,
                ctx->b_lo, ctx->b_hi);
        return BTE_EINVAL;
    }
    if (ctx->begun) return BTE_ESTATE;
    return BTE_OK;
}

bte_status bte_get_intensity(const bte_ctx *ctx, int32_t b_lo, int32_t b_hi, double *I) {
    if (!ctx || !I) return BTE_EINVAL;
    STATUS_TRY(check_rows(ctx, b_lo, b_hi));
    CUDA_TRY(const_cast<bte_ctx *>(ctx), cudaSetDevice(ctx->device));
    for (int32_t b = b_lo; b < b_hi; ++b) {
        const double *slab = ctx->pool_cells + (int64_t)ctx->cur_slot[b - ctx->b_lo] * ctx->slab_elems;
        STATUS_TRY(rows_to_host(ctx, slab, ctx->ps, ctx->nd, I + (int64_t)(b - b_lo) * ctx->nd * ctx->nc));
    }
    return BTE_OK;
}

bte_status bte_set_intensity(bte_ctx *ctx, int32_t b_lo, int32_t b_hi, const double *I) {
    if (!ctx || !I) return BTE_EINVAL;
    STATUS_TRY(check_rows(ctx, b_lo, b_hi));
    CUDA_TRY(ctx, cudaSetDevice(ctx->device));
    for (int32_t b = b_lo; b < b_hi; ++b) {
        double *slab = ctx->pool_cells + (int64_t)ctx->cur_slot[b - ctx->b_lo] * ctx->slab_elems;
        STATUS_TRY(rows_from_host(ctx, I + (int64_t)(b - b_lo) * ctx->nd * ctx->nc, ctx->ps, ctx->nd, slab));
    }
    CUDA_TRY(ctx, cudaStreamSynchronize(ctx->stream));
    return BTE_OK;
}

bte_status bte_solve_temperature(bte_ctx *ctx) {
    if (!ctx) return BTE_EINVAL;
    if (ctx->begun) return BTE_ESTATE;
    if (ctx->G > 1 && !ctx->have_comm)
        return set_err(&ctx->err, "world > 1 without a communicator: cannot reduce the energy"), BTE_ESTATE;
    CUDA_TRY(ctx, cudaSetDevice(ctx->device));
    STATUS_TRY(upload_cur_slots(ctx));
    const bool law_r2 = ctx->td && ctx->opt.temp_rule == 0;  // weights at the kept rate temperature
    bte::energy_kernel<<<(ctx->nc + 31) / 32, 32 * bte::kSumSlotWarps, 0, ctx->stream>>>(
        ctx->pool_cells, ctx->d_cur_slot, ctx->slab_elems, ctx->ps, ctx->nb_loc, ctx->nd, ctx->nc, ctx->dirs, ctx->cw_loc,
        law_r2 ? rate_half(ctx, ctx->rsel) : nullptr, ctx->td ? ctx->d_inv_v + ctx->b_lo : nullptr, ctx->E);
    CUDA_TRY(ctx, cudaGetLastError());
    STATUS_TRY(allreduce_E(ctx));
    STATUS_TRY(run_newton(ctx, ctx->E, /*step=*/false));
    STATUS_TRY(check_newton(ctx));
    if (ctx->td) {  // the dt bound follows the hottest cell of a state set from outside
        std::vector<double> T(ctx->nc);
        CUDA_TRY(ctx, cudaMemcpy(T.data(), ctx->T, ctx->nc * sizeof(double), cudaMemcpyDeviceToHost));
        for (double t : T) ctx->t_hi = std::max(ctx->t_hi, t);
        update_dt_bound(ctx);
    }
    return BTE_OK;
}

// Temperature of the current state under another rule (N4): energy reduction
// with that rule's weights, all-reduce, Newton (R3: one step) from the current
// T into scratch; the state (T, I0, rates) is not touched.
bte_status bte_get_temperature_rule(const bte_ctx *cctx, int32_t rule, double *T) {
    if (!cctx || !T) return BTE_EINVAL;
    bte_ctx *ctx = const_cast<bte_ctx *>(cctx);
    if (rule < 0 || rule > 2) return set_err(&ctx->err, "rule must be 0, 1 or 2"), BTE_EINVAL;
    if (ctx->begun) return BTE_ESTATE;
    if (ctx->G > 1 && !ctx->have_comm)
        return set_err(&ctx->err, "world > 1 without a communicator: cannot reduce the energy"), BTE_ESTATE;
    CUDA_TRY(ctx, cudaSetDevice(ctx->device));
    if (!ctx->E2) {
        STATUS_TRY(dalloc(ctx, &ctx->E2, (size_t)ctx->nc));
        STATUS_TRY(dalloc(ctx, &ctx->T2, (size_t)ctx->nc));
        STATUS_TRY(dalloc(ctx, &ctx->cw_diag, (size_t)ctx->nb));
    }
    std::vector<double> w(ctx->nb);
    bool any = false;
    for (int b = 0; b < ctx->nb; ++b) {
        w[b] = rule != 0 ? 1.0 / ctx->h_vg_all[b] : ctx->h_inv_tau_all[b] / ctx->h_vg_all[b];
        any |= w[b] > 0.0 || (ctx->td && ctx->h_rb[b] > 0.0);
    }
    if (!any) return set_err(&ctx->err, "all temperature weights are zero under rule %d", rule), BTE_EINVAL;
    CUDA_TRY(ctx, cudaMemcpyAsync(ctx->cw_diag, w.data(), ctx->nb * sizeof(double), cudaMemcpyHostToDevice,
                                  ctx->stream));
    STATUS_TRY(upload_cur_slots(ctx));
    const bool law_r2 = ctx->td && rule == 0;
    bte::energy_kernel<<<(ctx->nc + 31) / 32, 32 * bte::kSumSlotWarps, 0, ctx->stream>>>(
        ctx->pool_cells, ctx->d_cur_slot, ctx->slab_elems, ctx->ps, ctx->nb_loc, ctx->nd, ctx->nc, ctx->dirs,
        ctx->cw_diag + ctx->b_lo, law_r2 ? rate_half(ctx, ctx->rsel) : nullptr,
        ctx->td ? ctx->d_inv_v + ctx->b_lo : nullptr, ctx->E2);
    CUDA_TRY(ctx, cudaGetLastError());
    STATUS_TRY(allreduce_E(ctx, ctx->E2));
    bte::NewtonParams q{};
    q.nc = ctx->nc;
    q.nb = ctx->nb;
    q.E = ctx->E2;
    q.T = ctx->T;
    q.T_out = ctx->T2;
    q.Cb = ctx->Cb;
    q.theta = ctx->theta;
    q.cw = ctx->cw_diag;
    q.W = ctx->W;
    q.rtol = ctx->opt.newton_rtol;
    q.racc = std::max(0.01 * ctx->opt.newton_rtol, 16.0 * DBL_EPSILON);
    q.maxit = ctx->opt.newton_max_iter;
    q.iter_max = ctx->d_iter_max;
    q.fail = ctx->d_fail;
    q.single = rule == 2;
    if (ctx->td) {
        q.td = 1;
        q.tr_step = 0;
        q.r2 = rule == 0;
        q.ra = ctx->d_ra;
        q.rb = ctx->d_rb;
        q.rth = ctx->d_rth;
        q.inv_v = ctx->d_inv_v;
        q.Tr = ctx->Tr;
    }
    STATUS_TRY(launch_newton_cells(ctx, q));
    STATUS_TRY(check_newton(ctx));
    return rows_to_host(ctx, ctx->T2, ctx->nc, 1, T);
}

bte_status bte_set_equilibrium(bte_ctx *ctx, const double *T) {
    if (!ctx || !T) return BTE_EINVAL;
    if (ctx->begun) return BTE_ESTATE;
    CUDA_TRY(ctx, cudaSetDevice(ctx->device));
    for (int32_t c = 0; c < ctx->nc; ++c)
        if (!(T[c] > 0.0) || !std::isfinite(T[c])) return set_err(&ctx->err, "T[%d] must be > 0", c), BTE_EINVAL;
    STATUS_TRY(rows_from_host(ctx, T, ctx->nc, 1, ctx->T));
    STATUS_TRY(refresh_i0(ctx));
    if (ctx->td) {
        for (int32_t c = 0; c < ctx->nc; ++c) ctx->t_hi = std::max(ctx->t_hi, T[c]);
        update_dt_bound(ctx);
    }
    STATUS_TRY(upload_cur_slots(ctx));
    const int tb = 256;
    bte::equilibrium_kernel<<<dim3(std::min<int64_t>(4096, ((int64_t)ctx->nd * ctx->nc + tb - 1) / tb), ctx->nb_loc),
                              tb, 0, ctx->stream>>>(ctx->pool_cells, ctx->d_cur_slot, ctx->slab_elems, ctx->ps, ctx->nd,
                                                    ctx->nc, ctx->i0);
    CUDA_TRY(ctx, cudaGetLastError());
    CUDA_TRY(ctx, cudaStreamSynchronize(ctx->stream));
    return BTE_OK;
}

bte_status bte_get_stats(const bte_ctx *ctx, bte_stats *st) {
    if (!ctx || !st) return BTE_EINVAL;
    *st = ctx->st;
    st->dir_chunks = ctx->dir_chunks;
    st->flux_variant = ctx->box ? 6 : ctx->tma ? (!ctx->paired ? 7 : ctx->uniform_g ? 4 : 3) : 0;
    return BTE_OK;
}

bte_status bte_reset_stats(bte_ctx *ctx) {
    if (!ctx) return BTE_EINVAL;
    const bte_stats keep = ctx->st;
    std::memset(&ctx->st, 0, sizeof ctx->st);
    ctx->st.spare_slabs = keep.spare_slabs;
    ctx->st.n_interior_cells = keep.n_interior_cells;
    ctx->st.band_group = keep.band_group;
    ctx->st.block_threads = keep.block_threads;
    ctx->st.halo_bytes = keep.halo_bytes;
    return BTE_OK;
}

}  // extern "C"
