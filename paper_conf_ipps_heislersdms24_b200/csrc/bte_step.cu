// bte_step.cu -- the explicit step (see bte_internal.h): flux + relaxation +
// energy partial launches (Eq. 3, 5, 6; L412-418), the temperature solve
// (L407-418, L555-561), the device-side stop after a failed solve, the
// 2-step CUDA graph, bte_step and the split step.
#include "bte_internal.h"
#include <cfloat>

namespace bte_host {


// ------------------------------------------------------------- profiling
void ev_mark(bte_ctx *ctx, int phase, bool begin) {
    if (!(ctx->opt.flags & BTE_FLAG_PROFILE)) return;
    if (begin) {
        PhaseEvent pe;
        if (!ctx->ev_pool.empty()) {
            pe = ctx->ev_pool.back();
            ctx->ev_pool.pop_back();
        } else {
            cudaEventCreate(&pe.a);
            cudaEventCreate(&pe.b);
        }
        pe.phase = phase;
        cudaEventRecord(pe.a, ctx->stream);
        ctx->ev_live.push_back(pe);
    } else {
        cudaEventRecord(ctx->ev_live.back().b, ctx->stream);
    }
}

void ev_collect(bte_ctx *ctx) {  // after a stream sync
    if (ctx->ev_live.empty()) return;
    float total = 0.f;
    cudaEventElapsedTime(&total, ctx->ev_live.front().a, ctx->ev_live.back().b);
    ctx->st.ms_total += total;
    for (auto &pe : ctx->ev_live) {
        float ms = 0.f;
        cudaEventElapsedTime(&ms, pe.a, pe.b);
        double *dst = pe.phase == kPhFlux ? &ctx->st.ms_flux_interior
                      : pe.phase == kPhAllreduce ? &ctx->st.ms_allreduce
                      : pe.phase == kPhHalo      ? &ctx->st.ms_halo
                                                 : &ctx->st.ms_newton;
        *dst += ms;
        ctx->ev_pool.push_back(pe);
    }
    ctx->ev_live.clear();
}

// Flux + relaxation + energy partials for all local band-rows: per band batch
// of <= n_spare rows, one launch per segment of full band groups, reading the
// current slabs and writing the spare ones, which then become current (double
// buffering when n_spare == nb_loc, slab rotation otherwise).
// Box path: one launch per band batch; a CTA = (32 x 8 x L cell block,
// nbb band-rows, box_oc orbits), one energy slot per (band batch, orbit chunk).
bte_status run_flux_box(bte_ctx *ctx, double dt) {
    bte::BoxParams p{};
    p.n0 = ctx->bn[0];
    p.n1 = ctx->bn[1];
    p.n2 = ctx->bz_t;  // tensor layers (z-slab partition: + halo layers)
    p.zlo = ctx->bz_lo;
    p.nown = ctx->bn[2];
    p.L = ctx->box_L;
    p.n_orb = ctx->n_orb;
    p.nc = ctx->nc;
    p.stages = ctx->box_stages;
    p.zside[0] = ctx->bzside[0];
    p.zside[1] = ctx->bzside[1];
    p.rsel_cur = ctx->rsel;
    p.rsel_next = ctx->rate_now ? ctx->rsel : 1 - ctx->rsel;  // (R2 weights of this step's energy)
    p.rate_r2 = ctx->opt.temp_rule == 0;
    p.dt = dt;
    for (int a = 0; a < 3; ++a) p.g[a] = ctx->bgeo[a];
    p.orb = ctx->orb;
    p.dirs = ctx->dirs_box;
    p.part = ctx->part;
    p.pool = ctx->pool;
    p.slab_elems = ctx->slab_elems;
    p.ps = ctx->ps;
    p.fail = ctx->d_fail;
    p.halt = ctx->d_halt;
    const size_t smem = box_smem(ctx);
    int slot = 0;
    for (int l0 = 0; l0 < ctx->nb_loc; l0 += ctx->n_spare) {
        const int nbl = std::min(ctx->n_spare, ctx->nb_loc - l0);
        const BoxPlan bp = plan_box(ctx, nbl);
        p.tiles0 = bp.tiles0;
        p.tiles1 = bp.tiles1;
        p.zranges = bp.zranges;
        p.n_chunks = bp.n_chunks;
        p.orb_chunk = bp.oc;
        p.nbb = bp.nbb;
        p.n_slices = bp.n_batches * bp.n_chunks;
        p.nbl = nbl;
        p.band0 = l0;
        p.slot0 = slot;
        for (int k = 0; k < nbl; ++k) {
            const int b = l0 + k;
            p.in_slab[k] = ctx->cur_slot[b];
            p.out_slab[k] = ctx->spare_slot[k];
            p.dtit[k] = dt * ctx->h_inv_tau[b];
            p.kv[k] = dt * ctx->h_vg[b];
            p.cw[k] = ctx->h_cw[b];
            p.inv_v[k] = 1.0 / ctx->h_vg[b];
        }
        ctx->dir_chunks = bp.n_chunks;
        ctx->st.band_group = bp.nbb;
        const int64_t items = (int64_t)bp.tiles0 * bp.tiles1 * bp.zranges * p.n_slices;
        if (items > INT32_MAX) return set_err(&ctx->err, "box kernel: %lld work items", (long long)items), BTE_EINVAL;
        const dim3 grid((unsigned)items);
        ev_mark(ctx, kPhFlux, true);
        box_kernel(ctx)<<<grid, dim3(bte::kBoxThreads), smem, ctx->stream>>>(p, ctx->tm_in, ctx->tm_out, ctx->tm_i0,
                                                                           ctx->tm_side, ctx->tm_rate);
        ev_mark(ctx, kPhFlux, false);
        ctx->st.kernel_launches++;
        ctx->st.flux_launches++;
        slot += p.n_slices;
        CUDA_TRY(ctx, cudaGetLastError());
        for (int k = 0; k < nbl; ++k) std::swap(ctx->cur_slot[l0 + k], ctx->spare_slot[k]);
    }
    ctx->n_slots_step = slot;
    return BTE_OK;
}

bte_status run_flux(bte_ctx *ctx, double dt) {
    if (ctx->box) return run_flux_box(ctx, dt);
    bte::FluxParams p{};
    p.nc = ctx->nc;
    p.ps = ctx->ps;
    p.nd = ctx->nd;
    p.i0 = ctx->i0;
    p.part = ctx->part;
    p.nbr = ctx->nbr;
    p.nbm = ctx->nbm;
    p.gx = ctx->gx;
    p.gy = ctx->gy;
    p.gz = ctx->gz;
    std::memcpy(p.gu, ctx->gu, sizeof p.gu);
    p.fcode = ctx->fcode;
    p.fcode8 = ctx->fcode8;
    p.i0w = ctx->i0w;
    p.n_iso = ctx->n_iso;
    p.refl = ctx->refl;
    p.dirs = ctx->dirs;
    p.dt = dt;
    p.hl_off = ctx->hl_off;
    p.hl_cell = ctx->hl_cell;
    p.hl_pos = ctx->hl_pos;
    p.bl_off = ctx->bl_off;
    p.bl_col = ctx->bl_col;
    p.bl_cls = ctx->bl_cls;
    p.bl_pos = ctx->bl_pos;
    p.sidx = ctx->sidx;
    p.hstride = ctx->hstride;
    p.fail = ctx->d_fail;
    p.halt = ctx->d_halt;
    if (ctx->td) {
        p.rate_cur = rate_half(ctx, ctx->rsel);
        p.rate_next = rate_half(ctx, ctx->rate_now ? ctx->rsel : 1 - ctx->rsel);
        p.rate_r2 = ctx->opt.temp_rule == 0;
    }
    int slot = 0;
    const dim3 block(ctx->block);
    for (int l0 = 0; l0 < ctx->nb_loc; l0 += ctx->n_spare) {
        const int nbl_batch = std::min(ctx->n_spare, ctx->nb_loc - l0);
        for (const Segment &sg : segments(ctx, nbl_batch)) {
            const FluxLaunch fn =
                pick_flux(ctx->dim, ctx->mf_t, sg.bg, ctx->paired, ctx->uniform_g, ctx->tma);
            const LaunchPlan lp = plan_launch(ctx, sg.nbl, sg.bg);
            p.nbl = sg.nbl;
            p.band0 = l0 + sg.off;
            p.dchunk = lp.dchunk;
            p.n_dchunks = lp.n_dch;
            p.slot0 = slot;
            for (int k = 0; k < sg.nbl; ++k) {
                const int b = l0 + sg.off + k;  // rank-local band-row
                p.in_ptr[k] = ctx->pool_cells + (int64_t)ctx->cur_slot[b] * ctx->slab_elems;
                p.out_ptr[k] = ctx->pool_cells + (int64_t)ctx->spare_slot[sg.off + k] * ctx->slab_elems;
                p.dtit[k] = dt * ctx->h_inv_tau[b];
                p.kv[k] = dt * ctx->h_vg[b];
                p.cw[k] = ctx->h_cw[b];
                p.inv_v[k] = 1.0 / ctx->h_vg[b];
            }
            if (sg.off == 0) ctx->dir_chunks = lp.n_dch;
            const dim3 grid((ctx->nc + ctx->block - 1) / ctx->block, lp.groups * lp.n_dch);
            ev_mark(ctx, kPhFlux, true);
            CUDA_TRY(ctx, fn(grid, block, ctx->stream, p));
            ev_mark(ctx, kPhFlux, false);
            ctx->st.kernel_launches++;
            ctx->st.flux_launches++;
            slot += lp.groups * lp.n_dch;
        }
        CUDA_TRY(ctx, cudaGetLastError());
        for (int k = 0; k < nbl_batch; ++k) std::swap(ctx->cur_slot[l0 + k], ctx->spare_slot[k]);
    }
    ctx->n_slots_step = slot;
    return BTE_OK;
}

// The step's temperature solve, one kernel when this rank holds every band-row:
// the slot sum E (in sum_slots_kernel's order, bit for bit, unless E was reduced
// already), the per-cell solve (the first evaluation of g from the stored I0
// table, Householder steps, the accepting evaluation storing the new I0 rows)
// and the epilogue (T, Tr, rates; I0 only where not stored).  Small meshes (fewer
// cells than ~8 warps of threads per SM) take a group of 16 lanes per cell
// (newton_lanes_kernel), larger ones one thread per cell (newton_kernel).
// Measured on B200: C3 (14,400 cells) 0.066 ms per step (round 1) -> 0.031;
// C4 (131,072 cells) 0.155 -> ~0.07.  Band-sharded ranks (a chunk of cells for
// all rows, the I0 of local rows only) solve into Tg; newton_finish_kernel
// completes the step after the all-gather.  Re-solves of the current state
// (step = false) use newton_kernel with its own epilogue.
// Lanes per cell of the step's solve: 0 = thread per cell (newton_kernel), else
// a group of G lanes per cell (newton_lanes_kernel).
int newton_lanes(const bte_ctx *ctx, int ncells) {
    if (ctx->newton_mode) return ctx->newton_mode == 2 ? 0 : ctx->newton_mode;  // (BTE_NEWTON: tests / sweeps)
    if (ncells >= 32 * 8 * ctx->sm_count) return 0;
    // the most lanes (8 .. 32) that keep ~1,600 threads per SM (measured on B200, step
    // solve: C3's 14,400 cells 16 lanes 0.031 ms, 8: 0.034, 32: 0.043; C3t's 28,800
    // cells 8 lanes 0.052 ms, 16: 0.058, 32: 0.073)
    int g = 32;
    while (g > 8 && (int64_t)ncells * g > (int64_t)1600 * ctx->sm_count) g /= 2;
    return g;
}
bool warp_newton(const bte_ctx *ctx, int ncells) { return newton_lanes(ctx, ncells) > 0; }

// Band constants in shared memory: C, theta, c_b (+ the four rate-law arrays).
size_t newton_smem(const bte_ctx *ctx) {
    return (size_t)(8 * ctx->nb + 4 * ctx->n_terms) * sizeof(double) + (size_t)ctx->nb * sizeof(int32_t);
}

// Thread-per-cell solve over q.nc cells (block 0 counts the step when q.done).
bte_status launch_newton_cells(bte_ctx *ctx, const bte::NewtonParams &q) {
    if (q.nc <= 0) return BTE_OK;
    const int tb = 128;
    CUDA_TRY(ctx, ensure_smem((const void *)bte::newton_kernel, newton_smem(ctx)));
    bte::newton_kernel<<<(q.nc + tb - 1) / tb, tb, newton_smem(ctx), ctx->stream>>>(q);
    ctx->st.kernel_launches++;
    CUDA_TRY(ctx, cudaGetLastError());
    return BTE_OK;
}

// Group-of-lanes solve: G lanes per cell, R = band-rows per lane (the smallest
// power of two >= nb / G).
template <int G, int R>
bte_status launch_newton_lanes_gr(bte_ctx *ctx, const bte::NewtonParams &q) {
    CUDA_TRY(ctx, ensure_smem((const void *)bte::newton_lanes_kernel<G, R>, newton_smem(ctx)));
    const int64_t threads = (int64_t)q.nc * G;
    bte::newton_lanes_kernel<G, R><<<(unsigned)((threads + 255) / 256), 256, newton_smem(ctx), ctx->stream>>>(q);
    ctx->st.kernel_launches++;
    CUDA_TRY(ctx, cudaGetLastError());
    return BTE_OK;
}

template <int G>
bte_status launch_newton_lanes_g(bte_ctx *ctx, const bte::NewtonParams &q) {
    const int r = ((q.n_terms > 0 ? q.n_terms : ctx->nb) + G - 1) / G;
    if (r <= 2) return launch_newton_lanes_gr<G, 2>(ctx, q);
    if (r <= 4) return launch_newton_lanes_gr<G, 4>(ctx, q);
    if (r <= 8) return launch_newton_lanes_gr<G, 8>(ctx, q);
    if (r <= 16) return launch_newton_lanes_gr<G, 16>(ctx, q);
    if (G == 32) return launch_newton_lanes_gr<G, 32>(ctx, q);
    return set_err(&ctx->err, "%d band-rows: too many for %d lanes per cell", ctx->nb, G), BTE_EINVAL;
}

bte_status launch_newton_warp(bte_ctx *ctx, const bte::NewtonParams &q) {
    if (q.nc <= 0) return BTE_OK;
    static_assert(bte::kMaxBands <= 32 * 32, "group solve: at most 32 terms per lane");
    const int n = q.n_terms > 0 ? q.n_terms : ctx->nb;  // terms a cell's solve sums
    switch (newton_lanes(ctx, q.nc)) {
        case 4: return n <= 64 ? launch_newton_lanes_g<4>(ctx, q) : launch_newton_lanes_g<32>(ctx, q);
        case 8: return n <= 128 ? launch_newton_lanes_g<8>(ctx, q) : launch_newton_lanes_g<32>(ctx, q);
        case 16: return n <= 256 ? launch_newton_lanes_g<16>(ctx, q) : launch_newton_lanes_g<32>(ctx, q);
        default: return launch_newton_lanes_g<32>(ctx, q);
    }
}

bte_status run_newton(bte_ctx *ctx, const double *E_or_null, bool step) {
    ev_mark(ctx, kPhNewton, true);
    if (step) {  // E (the slot sum) -> the solve into Tg -> the epilogue (T, Tr, I0, rates) in parallel
        if (warp_newton(ctx, ctx->nc) && ctx->nb_loc == ctx->nb && newton_lanes(ctx, ctx->nc) >= bte::kSumSlotWarps) {
            // one kernel: the slot sum (unless E is given), the group-of-lanes solve and
            // its epilogue (C3: 3 launches -> 1)
            bte::NewtonParams q = newton_params(ctx, E_or_null, true);
            q.done = ctx->d_done;
            STATUS_TRY(launch_newton_warp(ctx, q));
            ev_mark(ctx, kPhNewton, false);
            if (ctx->td && !ctx->rate_now) ctx->rsel = 1 - ctx->rsel;
            return BTE_OK;
        }
        if (!warp_newton(ctx, ctx->nc)) {  // one thread per cell: slot sum, solve and epilogue in one kernel
            bte::NewtonParams q = newton_params(ctx, E_or_null, true);
            q.done = ctx->d_done;
            STATUS_TRY(launch_newton_cells(ctx, q));
            ev_mark(ctx, kPhNewton, false);
            if (ctx->td && !ctx->rate_now) ctx->rsel = 1 - ctx->rsel;
            return BTE_OK;
        }
        if (!E_or_null) {
            STATUS_TRY(reduce_slots(ctx));
            E_or_null = ctx->E;
        }
        bte::NewtonParams q = newton_params(ctx, E_or_null, true);
        if (warp_newton(ctx, ctx->nc)) {  // solve into Tg, then the epilogue over (row, cell)
            q.T_out = ctx->Tg;
            q.neg_fail = 1;
            if (q.spec) q.fresh = ctx->fresh;
            STATUS_TRY(launch_newton_warp(ctx, q));
            STATUS_TRY(newton_finish(ctx, q.fresh));  // (counts the step)
        } else {  // one thread per cell, epilogue in the same thread (C4: 0.13 vs 0.16 ms with the finish)
            q.done = ctx->d_done;
            STATUS_TRY(launch_newton_cells(ctx, q));
        }
        ev_mark(ctx, kPhNewton, false);
        if (ctx->td && !ctx->rate_now) ctx->rsel = 1 - ctx->rsel;
        return BTE_OK;
    }
    // a re-solve of the current state: one thread per cell, epilogue in place
    bte::NewtonParams q = newton_params(ctx, E_or_null, false);
    STATUS_TRY(launch_newton_cells(ctx, q));
    ev_mark(ctx, kPhNewton, false);
    return BTE_OK;
}

bte::NewtonParams newton_params(bte_ctx *ctx, const double *E_or_null, bool step) {
    bte::NewtonParams q{};
    if (ctx->td) {
        q.td = 1;
        q.tr_step = step;
        q.r2 = ctx->opt.temp_rule == 0;
        q.ra = ctx->d_ra;
        q.rb = ctx->d_rb;
        q.rth = ctx->d_rth;
        q.inv_v = ctx->d_inv_v;
        q.Tr = ctx->Tr;
        q.rate_out = rate_half(ctx, (step || ctx->rate_now) ? ctx->rsel : 1 - ctx->rsel);
        q.tr_now = ctx->rate_now;
    }
    q.nc = ctx->nc;
    q.nb = ctx->nb;
    q.n_slots = ctx->n_slots_step;
    q.part = ctx->part;
    q.E = E_or_null;
    q.T = ctx->T;
    q.i0 = ctx->i0;
    q.b_lo = ctx->b_lo;
    q.nb_loc = ctx->nb_loc;
    q.Cb = ctx->Cb;
    q.theta = ctx->theta;
    q.cw = ctx->cw_all;
    q.W = ctx->W;
    q.rtol = ctx->opt.newton_rtol;
    q.racc = std::max(0.01 * ctx->opt.newton_rtol, 16.0 * DBL_EPSILON);
    q.maxit = ctx->opt.newton_max_iter;
    q.iter_max = ctx->d_iter_max;
    q.fail = ctx->d_fail;
    q.single = ctx->opt.temp_rule == 2;
    if (step) q.halt = ctx->d_halt;  // (a step's solve: no-op after a failure earlier in the call)
    if (ctx->nb_loc == ctx->nb) {  // this rank's I0 table holds every row at the current T
        q.i0_t0 = ctx->i0;
        q.nc_tab = ctx->nc;
        q.spec = 1;  // (the accepting evaluation stores the rows' I0: no separate refresh)
    }
    q.n_terms = ctx->n_terms;
    q.t_th = ctx->t_th;
    q.t_k = ctx->t_k;
    q.t_ic = ctx->t_ic;
    q.t_rep = ctx->t_rep;
    q.t_nrow = ctx->t_nrow;
    return q;
}

bte_status reduce_slots(bte_ctx *ctx) {
    bte::sum_slots_kernel<<<(ctx->nc + 31) / 32, 32 * bte::kSumSlotWarps, 0, ctx->stream>>>(
        ctx->part, ctx->n_slots_step, ctx->nc, ctx->E, ctx->d_halt);
    ctx->st.kernel_launches++;
    CUDA_TRY(ctx, cudaGetLastError());
    return BTE_OK;
}


// T <- Tg (a negative entry marks a failed cell: flag, keep T^n), Tr <- T^n,
// I0 (unless fresh[c]: stored by the solve) and the rate table of the local rows at the new T.
bte_status newton_finish(bte_ctx *ctx, const int8_t *fresh) {
    const int64_t n = (int64_t)ctx->nc * ctx->nb_loc;
    bte::newton_finish_kernel<<<(unsigned)((n + 255) / 256), 256, 0, ctx->stream>>>(
        ctx->Tg, ctx->T, ctx->nc, ctx->b_lo, ctx->nb_loc, ctx->Cb, ctx->theta, ctx->i0, ctx->td, ctx->d_ra, ctx->d_rb,
        ctx->d_rth, ctx->Tr, ctx->td ? rate_half(ctx, ctx->rsel) : nullptr, ctx->d_fail, ctx->d_halt, ctx->d_done,
        ctx->rate_now ? 1 : 0, fresh);
    ctx->st.kernel_launches++;
    CUDA_TRY(ctx, cudaGetLastError());
    return BTE_OK;
}

// After the launches of a call: the failure flag and the steps that ran
// (*ran, since the last read); a failure resets the flags for the next call.
bte_status read_flags(bte_ctx *ctx, bool *failed, int64_t *ran) {
    int32_t h[4];
    CUDA_TRY(ctx, cudaMemcpyAsync(h, ctx->d_flags, 3 * sizeof(int32_t), cudaMemcpyDeviceToHost, ctx->stream));
    CUDA_TRY(ctx, cudaMemcpyAsync(&h[3], ctx->d_iter_max, sizeof(int32_t), cudaMemcpyDeviceToHost, ctx->stream));
    CUDA_TRY(ctx, cudaStreamSynchronize(ctx->stream));
    ev_collect(ctx);
    ctx->st.newton_iter_max = std::max(ctx->st.newton_iter_max, h[3]);
    *ran = (int64_t)(uint32_t)(h[2] - ctx->done_seen);
    ctx->done_seen = h[2];
    *failed = h[0] != 0;
    if (*failed) CUDA_TRY(ctx, cudaMemsetAsync(ctx->d_flags, 0, 2 * sizeof(int32_t), ctx->stream));  // fail, halt
    return BTE_OK;
}

bte_status check_newton(bte_ctx *ctx) {
    bool failed = false;
    int64_t ran = 0;
    STATUS_TRY(read_flags(ctx, &failed, &ran));
    if (failed) {
        set_err(&ctx->err, "temperature solve did not converge (non-positive or non-finite energy)");
        return BTE_ENOCONV;
    }
    return BTE_OK;
}

// Undo the host-side state advance of one step whose kernels were no-ops (a
// step after a failed solve): the slab swaps of run_flux in reverse batch
// order, and the rate-table halves.
void undo_step_rotation(bte_ctx *ctx) {
    int l0 = 0;
    std::vector<int> starts;
    for (; l0 < ctx->nb_loc; l0 += ctx->n_spare) starts.push_back(l0);
    for (auto it = starts.rbegin(); it != starts.rend(); ++it) {
        const int nbl = std::min(ctx->n_spare, ctx->nb_loc - *it);
        for (int k = 0; k < nbl; ++k) std::swap(ctx->cur_slot[*it + k], ctx->spare_slot[k]);
    }
    if (ctx->td && !ctx->rate_now) ctx->rsel = 1 - ctx->rsel;
}

// I0 of the current T; with the rate law also Tr = T and both rate halves at T
// (a state set to local equilibrium, bte_create / bte_set_equilibrium).
bte_status refresh_i0(bte_ctx *ctx) {
    const int tb = 256;
    const int gb = (ctx->nc + tb - 1) / tb;
    bte::i0_table_kernel<<<gb, tb, 0, ctx->stream>>>(ctx->T, ctx->nc, ctx->b_lo, ctx->nb_loc, ctx->Cb, ctx->theta,
                                                    ctx->i0);
    if (ctx->td) {
        CUDA_TRY(ctx, cudaMemcpyAsync(ctx->Tr, ctx->T, ctx->nc * sizeof(double), cudaMemcpyDeviceToDevice,
                                      ctx->stream));
        for (int h = 0; h < 2; ++h)
            bte::rate_table_kernel<<<gb, tb, 0, ctx->stream>>>(ctx->T, ctx->nc, ctx->b_lo, ctx->nb_loc, ctx->d_ra,
                                                              ctx->d_rb, ctx->d_rth, rate_half(ctx, h));
    }
    CUDA_TRY(ctx, cudaGetLastError());
    return BTE_OK;
}

// Positivity bound 1 / max_b (1/tau_b + v_b S_max); with the rate law the rates
// at t_hi (the max principle keeps T below it, P10).
void update_dt_bound(bte_ctx *ctx) {
    double rate = 0.0;
    for (int b = 0; b < ctx->nb; ++b) {
        const double r = ctx->td ? ctx->h_ra[b] + ctx->h_rb[b] * ctx->t_hi * std::exp(-ctx->h_rth[b] / ctx->t_hi)
                                 : ctx->h_inv_tau_all[b];
        rate = std::max(rate, r + ctx->h_vg_all[b] * ctx->s_max);
    }
    ctx->dt_bound = rate > 0.0 ? 1.0 / rate : INFINITY;
}

bte_status upload_cur_slots(bte_ctx *ctx) {
    CUDA_TRY(ctx, cudaMemcpyAsync(ctx->d_cur_slot, ctx->cur_slot.data(), ctx->nb_loc * sizeof(int32_t),
                                  cudaMemcpyHostToDevice, ctx->stream));
    return BTE_OK;
}

}  // namespace bte_host

using namespace bte_host;

extern "C" {


static bte_status check_dt(bte_ctx *ctx, double dt) {
    if (!(dt > 0.0) || !std::isfinite(dt)) return set_err(&ctx->err, "dt must be > 0 (got %g)", dt), BTE_EINVAL;
    if (dt > ctx->dt_bound * (1.0 + 1e-12))
        return set_err(&ctx->err, "dt = %.6g exceeds the positivity bound %.6g", dt, ctx->dt_bound), BTE_EINVAL;
    return BTE_OK;
}

// One explicit step (Eq. 2-3): halo exchange (cell partitioning), flux +
// relaxation + energy partials, the energy exchange and the temperature solve.
static bte_status one_step(bte_ctx *ctx, double dt) {
    STATUS_TRY(halo_exchange(ctx));
    STATUS_TRY(run_flux(ctx, dt));
    if (ctx->have_bcomm && ctx->shard_newton) {
        STATUS_TRY(shard_newton_step(ctx));
    } else if (ctx->have_bcomm) {
        ev_mark(ctx, kPhAllreduce, true);
        STATUS_TRY(reduce_slots(ctx));
        STATUS_TRY(allreduce_E(ctx));
        ev_mark(ctx, kPhAllreduce, false);
        STATUS_TRY(run_newton(ctx, ctx->E));
    } else {
        STATUS_TRY(run_newton(ctx, nullptr));
    }
    return BTE_OK;
}

// State key of the double-buffered pointers: which slab holds row 0 and which
// rate half is current (both flip every step).
static int graph_key(const bte_ctx *ctx) { return ctx->cur_slot[0] * 2 + ctx->rsel; }

// Capture two steps into a CUDA graph on the library stream (launch-bound
// small problems: one replay instead of ~8 launches).  Nothing runs during
// capture, so the host-side state the captured steps advance (slab rotation,
// rate halves, launch counters) is restored afterwards: a 2-step capture of a
// double-buffered state ends where it began anyway, and a failed capture must
// not leave it advanced.  A failure is recorded (ctx->err) and disables graphs
// for the context; the steps then run launch by launch.
static void capture_two_steps(bte_ctx *ctx, double dt) {
    if (ctx->gexec) {
        cudaGraphExecDestroy(ctx->gexec);
        ctx->gexec = nullptr;
    }
    const std::vector<int32_t> cur0 = ctx->cur_slot, spare0 = ctx->spare_slot;
    const int rsel0 = ctx->rsel, dch0 = ctx->dir_chunks, slots0 = ctx->n_slots_step;
    const int64_t l0 = ctx->st.kernel_launches, f0 = ctx->st.flux_launches;
    const int key = graph_key(ctx);
    cudaGraph_t g = nullptr;
    cudaError_t ce = cudaStreamBeginCapture(ctx->stream, cudaStreamCaptureModeThreadLocal);
    bte_status s1 = BTE_OK, s2 = BTE_OK;
    bool closed = false;
    if (ce == cudaSuccess) {
        s1 = one_step(ctx, dt);
        if (s1 == BTE_OK) s2 = one_step(ctx, dt);
        closed = graph_key(ctx) == key;  // (the rotation of two steps must close to replay)
        ce = cudaStreamEndCapture(ctx->stream, &g);
    }
    if (ce == cudaSuccess && s1 == BTE_OK && s2 == BTE_OK && g && closed)
        ce = cudaGraphInstantiate(&ctx->gexec, g, 0);
    if (g) cudaGraphDestroy(g);
    ctx->g_launches = ctx->st.kernel_launches - l0;
    ctx->g_flux = ctx->st.flux_launches - f0;
    ctx->st.kernel_launches = l0;
    ctx->st.flux_launches = f0;
    ctx->cur_slot = cur0;
    ctx->spare_slot = spare0;
    ctx->rsel = rsel0;
    ctx->dir_chunks = dch0;
    ctx->n_slots_step = slots0;
    if (ce != cudaSuccess || s1 != BTE_OK || s2 != BTE_OK || !closed || !ctx->gexec) {
        if (ctx->gexec) cudaGraphExecDestroy(ctx->gexec);
        ctx->gexec = nullptr;
        ctx->graphs_ok = false;
        cudaGetLastError();
        set_err(&ctx->err, "CUDA graph capture disabled (%s%s%s); stepping launch by launch",
                ce != cudaSuccess ? cudaGetErrorString(ce) : "",
                (s1 != BTE_OK || s2 != BTE_OK) ? " step failed under capture" : "",
                !closed ? " slab rotation does not close over two steps" : "");
        return;
    }
    ctx->g_key = key;
    ctx->g_dt = dt;
}

bte_status bte_step(bte_ctx *ctx, double dt, int64_t n) {
    if (!ctx) return BTE_EINVAL;
    if (ctx->begun) return set_err(&ctx->err, "split step in flight"), BTE_ESTATE;
    if (n < 0) return set_err(&ctx->err, "n < 0"), BTE_EINVAL;
    if (n == 0) return BTE_OK;
    if (ctx->opt.world > 1 && !ctx->have_comm)
        return set_err(&ctx->err, "world > 1 without a communicator: reduce the energy (and move the halo) with "
                                  "bte_step_begin / bte_get_energy / bte_set_energy / bte_step_finish "
                                  "(bte_halo_export / bte_halo_import)"), BTE_ESTATE;
    CUDA_TRY(ctx, cudaSetDevice(ctx->device));
    STATUS_TRY(sync_dt_bound(ctx));  // (collective with cell partitioning + the rate law)
    STATUS_TRY(check_dt(ctx, dt));
    const int64_t upd = (int64_t)ctx->nc * ctx->nd * ctx->nb_loc;
    int64_t s = 0;
    auto step1 = [&]() -> bte_status {
        STATUS_TRY(one_step(ctx, dt));
        ctx->st.steps++;
        ctx->st.updates += upd;
        ++s;
        return BTE_OK;
    };
    // CUDA graphs: double buffering, no per-phase events (BTE_NO_GRAPH=1 disables).  The
    // NCCL exchanges of band sharding / cell partitioning are captured too (NCCL supports
    // stream capture); every rank replays the same sequence of collectives.
    const bool no_graph_env = std::getenv("BTE_NO_GRAPH") != nullptr;
    const bool graphs = ctx->graphs_ok && !no_graph_env && n >= 4 && !(ctx->opt.flags & BTE_FLAG_PROFILE) &&
                        ctx->n_spare == ctx->nb_loc;
    if (graphs) {
        if (!ctx->gexec || ctx->g_dt != dt) {
            STATUS_TRY(step1());  // (first launches set the kernels' shared-memory attributes)
            capture_two_steps(ctx, dt);
        }
        if (ctx->gexec && graph_key(ctx) != ctx->g_key) STATUS_TRY(step1());
        for (; ctx->gexec && s + 2 <= n; s += 2) {
            CUDA_TRY(ctx, cudaGraphLaunch(ctx->gexec, ctx->stream));
            ctx->st.steps += 2;
            ctx->st.updates += 2 * upd;
            ctx->st.kernel_launches += ctx->g_launches;
            ctx->st.flux_launches += ctx->g_flux;
            ctx->st.graph_replays++;
        }
    }
    while (s < n) STATUS_TRY(step1());
    // A failed temperature solve in step k made steps k+1..n no-ops on the device
    // (bte_kernels.cuh: fail / halt): undo their host-side rotation so that the
    // state is the one at the end of the failing step (ENOCONV
    // "with the state at the failing step").
    bool failed = false;
    int64_t ran = 0;
    STATUS_TRY(read_flags(ctx, &failed, &ran));
    if (failed) {
        const int64_t skipped = std::max<int64_t>(0, n - ran);
        for (int64_t i = 0; i < skipped; ++i) undo_step_rotation(ctx);
        ctx->st.steps -= skipped;
        ctx->st.updates -= skipped * upd;
        STATUS_TRY(upload_cur_slots(ctx));
        CUDA_TRY(ctx, cudaStreamSynchronize(ctx->stream));
        set_err(&ctx->err, "temperature solve did not converge (non-positive or non-finite energy) in step %lld of "
                           "%lld; the state is the one at the end of that step (failed cells keep their previous T)",
                (long long)ran, (long long)n);
        return BTE_ENOCONV;
    }
    STATUS_TRY(upload_cur_slots(ctx));
    return BTE_OK;
}

bte_status bte_step_begin(bte_ctx *ctx, double dt) {
    if (!ctx) return BTE_EINVAL;
    if (ctx->begun) return set_err(&ctx->err, "split step already begun"), BTE_ESTATE;
    CUDA_TRY(ctx, cudaSetDevice(ctx->device));
    STATUS_TRY(sync_dt_bound(ctx));
    STATUS_TRY(check_dt(ctx, dt));
    if (ctx->have_comm) STATUS_TRY(halo_exchange(ctx));  // (no communicator: the caller imported the halo)
    STATUS_TRY(run_flux(ctx, dt));
    STATUS_TRY(reduce_slots(ctx));
    STATUS_TRY(upload_cur_slots(ctx));
    CUDA_TRY(ctx, cudaStreamSynchronize(ctx->stream));
    ctx->begun = true;
    return BTE_OK;
}

bte_status bte_step_finish(bte_ctx *ctx) {
    if (!ctx) return BTE_EINVAL;
    if (!ctx->begun) return set_err(&ctx->err, "bte_step_finish without bte_step_begin"), BTE_ESTATE;
    CUDA_TRY(ctx, cudaSetDevice(ctx->device));
    STATUS_TRY(run_newton(ctx, ctx->E));
    ctx->begun = false;
    ctx->st.steps++;
    ctx->st.updates += (int64_t)ctx->nc * ctx->nd * ctx->nb_loc;
    return check_newton(ctx);
}

}  // extern "C"
