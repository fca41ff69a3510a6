// bte_api.cu -- host runtime behind include/bte.h.
//
// Owns validation, the device layout (cell reorder, padded face slots,
// reflection maps, slab pool), launch planning, the per-step launch sequence,
// the NCCL energy all-reduce and the getters.  All arithmetic of the step runs
// in the kernels of bte_kernels.cuh; the host only moves data and plans.
#include "../../include/bte.h"
#include "bte_kernels.cuh"
#include "bte_nccl.h"

#include <algorithm>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <map>
#include <string>
#include <vector>

namespace {

// CODATA 2018 values (library's own copy; theta_b = hbar omega_b / kB).
constexpr double kHbar = 1.054571817e-34;
constexpr double kKb = 1.380649e-23;
constexpr int kMaxFaces = 8;

thread_local std::string g_err = "no error";

void set_err(std::string *dst, const char *fmt, ...) {
    char buf[1024];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    g_err = buf;
    if (dst) *dst = buf;
}

struct PhaseEvent {
    int phase;
    cudaEvent_t a, b;
};
enum Phase { kPhInterior = 0, kPhBoundary = 1, kPhAllreduce = 2, kPhNewton = 3 };

}  // namespace

struct bte_ctx {
    std::string err = "no error";
    bte_options opt{};
    int dim = 0, nd = 0, nb = 0, b_lo = 0, b_hi = 0, nb_loc = 0, mf = 0, mf_t = 0;
    int32_t nc = 0, n_int = 0;
    int device = 0;
    int sm_count = 148;
    double W = 0.0, s_max = 0.0, dt_bound = 0.0;
    // device state
    double *pool = nullptr;
    int64_t slab_elems = 0;
    int n_spare = 0;
    std::vector<int32_t> cur_slot, spare_slot;
    int32_t *d_cur_slot = nullptr;  // for energy/equilibrium kernels
    double *i0 = nullptr, *T = nullptr, *E = nullptr, *part = nullptr;
    int n_slots_step = 0;
    double *staging = nullptr;
    int64_t staging_elems = 0;
    int32_t *nbr = nullptr, *aux = nullptr, *refl = nullptr, *pos = nullptr;
    double *gx = nullptr, *gy = nullptr, *gz = nullptr;
    int8_t *kind = nullptr;
    double *i0w = nullptr, *twall = nullptr;
    int32_t n_iso = 0, n_refl = 0;
    double4 *dirs = nullptr;
    double *inv_tau = nullptr, *vg = nullptr, *cw_loc = nullptr;
    double *Cb = nullptr, *theta = nullptr, *cw_all = nullptr;
    int32_t *d_iter_max = nullptr, *d_fail = nullptr;
    unsigned long long *d_smax = nullptr;
    // launch plan
    int bg = 4, block = 256;
    int dir_chunks = 1;
    // execution
    cudaStream_t stream = nullptr;
    bool own_stream = false;
    bte::nccl::Comm comm{};
    bool have_comm = false;
    bool begun = false;  // split step in flight
    double begun_dt = 0.0;
    // stats
    bte_stats st{};
    std::vector<PhaseEvent> ev_live, ev_pool;
};

namespace {

#define CUDA_TRY(ctx, call)                                                                 \
    do {                                                                                    \
        cudaError_t e_ = (call);                                                            \
        if (e_ != cudaSuccess) {                                                            \
            set_err((ctx) ? &(ctx)->err : nullptr, "CUDA error %s at %s:%d: %s",            \
                    cudaGetErrorName(e_), __FILE__, __LINE__, cudaGetErrorString(e_));      \
            return e_ == cudaErrorMemoryAllocation ? BTE_ENOMEM : BTE_ECUDA;                \
        }                                                                                   \
    } while (0)

#define STATUS_TRY(call)              \
    do {                              \
        bte_status s_ = (call);       \
        if (s_ != BTE_OK) return s_;  \
    } while (0)

template <class T>
bte_status dalloc(bte_ctx *ctx, T **p, size_t n) {
    CUDA_TRY(ctx, cudaMalloc((void **)p, std::max<size_t>(n, 1) * sizeof(T)));
    return BTE_OK;
}

template <class T>
bte_status upload(bte_ctx *ctx, T **p, const std::vector<T> &h) {
    STATUS_TRY(dalloc(ctx, p, h.size()));
    if (!h.empty()) CUDA_TRY(ctx, cudaMemcpy(*p, h.data(), h.size() * sizeof(T), cudaMemcpyHostToDevice));
    return BTE_OK;
}

// ------------------------------------------------------------- template dispatch
using FluxLaunch = void (*)(bool, dim3, dim3, cudaStream_t, const bte::FluxParams &);

template <int DIM, int MF, int BG>
void flux_launch_t(bool bnd, dim3 g, dim3 b, cudaStream_t s, const bte::FluxParams &p) {
    if (bnd)
        bte::flux_kernel<DIM, MF, BG, true><<<g, b, 0, s>>>(p);
    else
        bte::flux_kernel<DIM, MF, BG, false><<<g, b, 0, s>>>(p);
}

template <int DIM, int MF>
FluxLaunch pick_bg(int bg) {
    switch (bg) {
        case 1: return flux_launch_t<DIM, MF, 1>;
        case 2: return flux_launch_t<DIM, MF, 2>;
        case 4: return flux_launch_t<DIM, MF, 4>;
        default: return flux_launch_t<DIM, MF, 8>;
    }
}

FluxLaunch pick_flux(int dim, int mf_t, int bg) {
    if (dim == 2) return mf_t == 4 ? pick_bg<2, 4>(bg) : pick_bg<2, 8>(bg);
    return mf_t == 6 ? pick_bg<3, 6>(bg) : pick_bg<3, 8>(bg);
}

int round_bg(int bg) { return bg <= 1 ? 1 : bg <= 2 ? 2 : bg <= 4 ? 4 : 8; }

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
        double *dst = pe.phase == kPhInterior   ? &ctx->st.ms_flux_interior
                      : pe.phase == kPhBoundary ? &ctx->st.ms_flux_boundary
                      : pe.phase == kPhAllreduce ? &ctx->st.ms_allreduce
                                                 : &ctx->st.ms_newton;
        *dst += ms;
        ctx->ev_pool.push_back(pe);
    }
    ctx->ev_live.clear();
}

// ------------------------------------------------------------- launch plan
struct LaunchPlan {
    int groups, n_dch, dchunk;
};

LaunchPlan plan_launch(const bte_ctx *ctx, int nbl, int cells) {
    LaunchPlan lp;
    lp.groups = (nbl + ctx->bg - 1) / ctx->bg;
    const int64_t target = (int64_t)ctx->sm_count * 2048 * 2;  // ~2 full waves of threads
    const int64_t have = std::max<int64_t>(1, (int64_t)cells * lp.groups);
    int n = (int)std::min<int64_t>(ctx->nd, std::max<int64_t>(1, (target + have - 1) / have));
    if (ctx->opt.flags & 0x100u) n = 1;  // (debug) force one chunk
    lp.dchunk = (ctx->nd + n - 1) / n;
    lp.n_dch = (ctx->nd + lp.dchunk - 1) / lp.dchunk;
    return lp;
}

// Flux + relaxation + energy partials for all local band-rows: one launch pair
// (interior, boundary) per band batch of <= n_spare rows, rotating slabs.
bte_status run_flux(bte_ctx *ctx, double dt) {
    bte::FluxParams p{};
    p.nc = ctx->nc;
    p.nd = ctx->nd;
    p.slab_elems = ctx->slab_elems;
    p.pool = ctx->pool;
    p.i0 = ctx->i0;
    p.part = ctx->part;
    p.nbr = ctx->nbr;
    p.gx = ctx->gx;
    p.gy = ctx->gy;
    p.gz = ctx->gz;
    p.kind = ctx->kind;
    p.aux = ctx->aux;
    p.refl = ctx->refl;
    p.i0w = ctx->i0w;
    p.n_iso = ctx->n_iso;
    p.dirs = ctx->dirs;
    p.inv_tau = ctx->inv_tau;
    p.vg = ctx->vg;
    p.cw = ctx->cw_loc;
    p.dt = dt;
    p.bg = ctx->bg;
    FluxLaunch fn = pick_flux(ctx->dim, ctx->mf_t, ctx->bg);
    int slot = 0;
    const int n_bnd = ctx->nc - ctx->n_int;
    for (int l0 = 0; l0 < ctx->nb_loc; l0 += ctx->n_spare) {
        const int nbl = std::min(ctx->n_spare, ctx->nb_loc - l0);
        p.nbl = nbl;
        p.band0 = l0;
        p.slot0 = slot;
        for (int k = 0; k < nbl; ++k) {
            p.in_slot[k] = ctx->cur_slot[l0 + k];
            p.out_slot[k] = ctx->spare_slot[k];
        }
        LaunchPlan lp = plan_launch(ctx, nbl, ctx->n_int > 0 ? ctx->n_int : n_bnd);
        p.dchunk = lp.dchunk;
        p.n_dchunks = lp.n_dch;
        ctx->dir_chunks = lp.n_dch;
        const dim3 block(ctx->block);
        if (ctx->n_int > 0) {
            p.cell_begin = 0;
            p.cell_end = ctx->n_int;
            dim3 grid((ctx->n_int + ctx->block - 1) / ctx->block, lp.groups * lp.n_dch);
            ev_mark(ctx, kPhInterior, true);
            fn(false, grid, block, ctx->stream, p);
            ev_mark(ctx, kPhInterior, false);
            ctx->st.kernel_launches++;
        }
        if (n_bnd > 0) {
            p.cell_begin = ctx->n_int;
            p.cell_end = ctx->nc;
            dim3 grid((n_bnd + ctx->block - 1) / ctx->block, lp.groups * lp.n_dch);
            ev_mark(ctx, kPhBoundary, true);
            fn(true, grid, block, ctx->stream, p);
            ev_mark(ctx, kPhBoundary, false);
            ctx->st.kernel_launches++;
        }
        CUDA_TRY(ctx, cudaGetLastError());
        slot += lp.groups * lp.n_dch;
        for (int k = 0; k < nbl; ++k) std::swap(ctx->cur_slot[l0 + k], ctx->spare_slot[k]);
    }
    ctx->n_slots_step = slot;
    return BTE_OK;
}

bte_status run_newton(bte_ctx *ctx, const double *E_or_null) {
    bte::NewtonParams q{};
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
    q.maxit = ctx->opt.newton_max_iter;
    q.iter_max = ctx->d_iter_max;
    q.fail = ctx->d_fail;
    const int tb = 128;
    ev_mark(ctx, kPhNewton, true);
    bte::newton_kernel<<<(ctx->nc + tb - 1) / tb, tb, 3 * ctx->nb * sizeof(double), ctx->stream>>>(q);
    ev_mark(ctx, kPhNewton, false);
    ctx->st.kernel_launches++;
    CUDA_TRY(ctx, cudaGetLastError());
    return BTE_OK;
}

bte_status allreduce_E(bte_ctx *ctx) {
    if (ctx->opt.world <= 1) return BTE_OK;
    std::string e;
    if (!bte::nccl::allreduce_sum_f64(ctx->comm, ctx->E, ctx->nc, ctx->stream, &e)) {
        set_err(&ctx->err, "NCCL all-reduce failed: %s", e.c_str());
        return BTE_ENCCL;
    }
    return BTE_OK;
}

bte_status reduce_slots(bte_ctx *ctx) {
    const int tb = 256;
    bte::sum_slots_kernel<<<(ctx->nc + tb - 1) / tb, tb, 0, ctx->stream>>>(ctx->part, ctx->n_slots_step,
                                                                           ctx->nc, ctx->E);
    ctx->st.kernel_launches++;
    CUDA_TRY(ctx, cudaGetLastError());
    return BTE_OK;
}

bte_status check_newton(bte_ctx *ctx) {
    int32_t h[2];
    CUDA_TRY(ctx, cudaMemcpyAsync(&h[0], ctx->d_fail, sizeof(int32_t), cudaMemcpyDeviceToHost, ctx->stream));
    CUDA_TRY(ctx, cudaMemcpyAsync(&h[1], ctx->d_iter_max, sizeof(int32_t), cudaMemcpyDeviceToHost, ctx->stream));
    CUDA_TRY(ctx, cudaStreamSynchronize(ctx->stream));
    ev_collect(ctx);
    ctx->st.newton_iter_max = std::max(ctx->st.newton_iter_max, h[1]);
    if (h[0]) {
        CUDA_TRY(ctx, cudaMemsetAsync(ctx->d_fail, 0, sizeof(int32_t), ctx->stream));
        set_err(&ctx->err, "temperature solve did not converge (non-positive or non-finite energy)");
        return BTE_ENOCONV;
    }
    return BTE_OK;
}

bte_status refresh_i0(bte_ctx *ctx) {
    const int tb = 256;
    bte::i0_table_kernel<<<(ctx->nc + tb - 1) / tb, tb, 0, ctx->stream>>>(ctx->T, ctx->nc, ctx->b_lo,
                                                                          ctx->nb_loc, ctx->Cb, ctx->theta,
                                                                          ctx->i0);
    CUDA_TRY(ctx, cudaGetLastError());
    return BTE_OK;
}

bte_status upload_cur_slots(bte_ctx *ctx) {
    CUDA_TRY(ctx, cudaMemcpyAsync(ctx->d_cur_slot, ctx->cur_slot.data(), ctx->nb_loc * sizeof(int32_t),
                                  cudaMemcpyHostToDevice, ctx->stream));
    return BTE_OK;
}

// ------------------------------------------------------------- validation
bool unit(const double *v, double tol) {
    const double n = std::sqrt(v[0] * v[0] + v[1] * v[1] + v[2] * v[2]);
    return std::fabs(n - 1.0) <= tol;
}

bte_status validate(const bte_mesh *m, const bte_bands *b, const bte_dirs *d, const bte_bcs *bc,
                    const bte_options *o) {
    if (!m || !b || !d || !bc || !o) return set_err(nullptr, "NULL argument"), BTE_EINVAL;
    if (m->dim != 2 && m->dim != 3) return set_err(nullptr, "dim must be 2 or 3 (got %d)", m->dim), BTE_EINVAL;
    if (m->n_cells <= 0 || m->n_cells >= (int64_t)1 << 31)
        return set_err(nullptr, "n_cells out of range"), BTE_EINVAL;
    if (!m->face_offsets || !m->face_nbr || !m->face_area || !m->face_normal || !m->cell_volume)
        return set_err(nullptr, "mesh array is NULL"), BTE_EINVAL;
    if (m->face_offsets[0] != 0) return set_err(nullptr, "face_offsets[0] must be 0"), BTE_EINVAL;
    for (int64_t c = 0; c < m->n_cells; ++c) {
        const int64_t nf = m->face_offsets[c + 1] - m->face_offsets[c];
        if (nf < 1 || nf > kMaxFaces)
            return set_err(nullptr, "cell %lld has %lld faces (1..8 supported)", (long long)c, (long long)nf),
                   BTE_EINVAL;
        if (!(m->cell_volume[c] > 0.0)) return set_err(nullptr, "cell %lld volume <= 0", (long long)c), BTE_EINVAL;
    }
    const int64_t nfaces = m->face_offsets[m->n_cells];
    for (int64_t f = 0; f < nfaces; ++f) {
        if (!(m->face_area[f] > 0.0)) return set_err(nullptr, "face %lld area <= 0", (long long)f), BTE_EINVAL;
        const double *n = m->face_normal + 3 * f;
        if (!unit(n, 1e-9)) return set_err(nullptr, "face %lld normal not unit", (long long)f), BTE_EINVAL;
        if (m->dim == 2 && n[2] != 0.0) return set_err(nullptr, "2-D mesh with n_z != 0 (face %lld)", (long long)f), BTE_EINVAL;
        const int64_t nb = m->face_nbr[f];
        if (nb >= m->n_cells) return set_err(nullptr, "face %lld neighbour out of range", (long long)f), BTE_EINVAL;
        if (nb < 0 && -1 - nb >= bc->n_bfaces)
            return set_err(nullptr, "face %lld boundary id out of range", (long long)f), BTE_EINVAL;
    }
    if (b->n_bands < 1 || !b->omega || !b->vg || !b->tau)
        return set_err(nullptr, "band table incomplete"), BTE_EINVAL;
    if (!b->i0_prefactor) return set_err(nullptr, "i0_prefactor (C_b) is required"), BTE_EINVAL;
    for (int i = 0; i < b->n_bands; ++i) {
        if (!(b->omega[i] > 0.0) || !(b->vg[i] > 0.0) || !(b->tau[i] > 0.0) || !(b->i0_prefactor[i] > 0.0))
            return set_err(nullptr, "band-row %d: omega, vg, tau, C must be > 0", i), BTE_EINVAL;
    }
    if (d->n_dirs < 1 || !d->s || !d->w) return set_err(nullptr, "direction set incomplete"), BTE_EINVAL;
    for (int i = 0; i < d->n_dirs; ++i) {
        if (!unit(d->s + 3 * i, 1e-9)) return set_err(nullptr, "direction %d not unit", i), BTE_EINVAL;
        if (!(d->w[i] > 0.0)) return set_err(nullptr, "direction %d weight <= 0", i), BTE_EINVAL;
    }
    for (int64_t f = 0; f < bc->n_bfaces; ++f) {
        if (bc->kind[f] != BTE_BC_ISOTHERMAL && bc->kind[f] != BTE_BC_SYMMETRY)
            return set_err(nullptr, "boundary face %lld: unknown kind %d", (long long)f, bc->kind[f]), BTE_EINVAL;
        if (bc->kind[f] == BTE_BC_ISOTHERMAL && !(bc->t_wall[f] > 0.0))
            return set_err(nullptr, "boundary face %lld: wall temperature <= 0", (long long)f), BTE_EINVAL;
    }
    if (o->temp_rule != 0 && o->temp_rule != 1) return set_err(nullptr, "temp_rule must be 0 or 1"), BTE_EINVAL;
    if (!(o->t_init > 0.0)) return set_err(nullptr, "t_init must be > 0"), BTE_EINVAL;
    if (o->world < 1 || o->rank < 0 || o->rank >= o->world) return set_err(nullptr, "bad rank/world"), BTE_EINVAL;
    if (!(o->newton_rtol > 0.0) || o->newton_max_iter < 1) return set_err(nullptr, "bad Newton controls"), BTE_EINVAL;
    return BTE_OK;
}

}  // namespace

// ============================================================= public API
extern "C" {

const char *bte_status_string(bte_status s) {
    switch (s) {
        case BTE_OK: return "BTE_OK";
        case BTE_EINVAL: return "BTE_EINVAL";
        case BTE_ENOMEM: return "BTE_ENOMEM";
        case BTE_ECUDA: return "BTE_ECUDA";
        case BTE_ENCCL: return "BTE_ENCCL";
        case BTE_ENOCONV: return "BTE_ENOCONV";
        case BTE_ESTATE: return "BTE_ESTATE";
    }
    return "BTE_UNKNOWN";
}

const char *bte_last_error(const bte_ctx *ctx) { return ctx ? ctx->err.c_str() : g_err.c_str(); }

bte_status bte_options_default(bte_options *o) {
    if (!o) return BTE_EINVAL;
    std::memset(o, 0, sizeof *o);
    o->t_init = 300.0;
    o->temp_rule = 0;
    o->newton_rtol = 1e-12;
    o->newton_max_iter = 50;
    o->rank = 0;
    o->world = 1;
    o->device = 0;
    return BTE_OK;
}

bte_status bte_nccl_unique_id(void *id128) {
    std::string e;
    if (!id128) return set_err(nullptr, "NULL id buffer"), BTE_EINVAL;
    if (!bte::nccl::unique_id(id128, &e)) return set_err(nullptr, "%s", e.c_str()), BTE_ENCCL;
    return BTE_OK;
}

void bte_destroy(bte_ctx *ctx) {
    if (!ctx) return;
    cudaSetDevice(ctx->device);
    if (ctx->stream) cudaStreamSynchronize(ctx->stream);
    if (ctx->have_comm) bte::nccl::destroy(ctx->comm);
    void *ptrs[] = {ctx->pool, ctx->d_cur_slot, ctx->i0, ctx->T, ctx->E, ctx->part, ctx->staging,
                    ctx->nbr, ctx->aux, ctx->refl, ctx->pos, ctx->gx, ctx->gy, ctx->gz, ctx->kind,
                    ctx->i0w, ctx->twall, ctx->dirs, ctx->inv_tau, ctx->vg, ctx->cw_loc, ctx->Cb,
                    ctx->theta, ctx->cw_all, ctx->d_iter_max, ctx->d_fail, ctx->d_smax};
    for (void *p : ptrs)
        if (p) cudaFree(p);
    for (auto &pe : ctx->ev_pool) cudaEventDestroy(pe.a), cudaEventDestroy(pe.b);
    for (auto &pe : ctx->ev_live) cudaEventDestroy(pe.a), cudaEventDestroy(pe.b);
    if (ctx->own_stream && ctx->stream) cudaStreamDestroy(ctx->stream);
    delete ctx;
}

bte_status bte_create(const bte_mesh *m, const bte_bands *bd, const bte_dirs *dr, const bte_bcs *bc,
                      const bte_options *o, bte_ctx **out) {
    if (!out) return set_err(nullptr, "NULL out"), BTE_EINVAL;
    *out = nullptr;
    STATUS_TRY(validate(m, bd, dr, bc, o));
    const int nd = dr->n_dirs, nb = bd->n_bands;
    const int64_t nc64 = m->n_cells;
    const int32_t nc = (int32_t)nc64;

    // --- temperature weights c_b and band constants
    std::vector<double> cw(nb), theta(nb), inv_tau(nb);
    bool any_w = false;
    for (int b = 0; b < nb; ++b) {
        inv_tau[b] = std::isinf(bd->tau[b]) ? 0.0 : 1.0 / bd->tau[b];
        cw[b] = o->temp_rule == 1 ? 1.0 / bd->vg[b] : (std::isinf(bd->tau[b]) ? 0.0 : 1.0 / (bd->vg[b] * bd->tau[b]));
        theta[b] = kHbar * bd->omega[b] / kKb;
        any_w |= cw[b] > 0.0;
    }
    if (!any_w) return set_err(nullptr, "all temperature weights are zero (temp_rule 0 with every tau = inf)"), BTE_EINVAL;

    // --- band sharding: rank g owns [floor(g nb/P), floor((g+1) nb/P))  (L760-775)
    const int b_lo = (int)((int64_t)o->rank * nb / o->world);
    const int b_hi = (int)((int64_t)(o->rank + 1) * nb / o->world);
    const int nb_loc = b_hi - b_lo;
    if (nb_loc < 1) return set_err(nullptr, "rank %d owns no band-row (n_bands %d < world %d)", o->rank, nb, o->world), BTE_EINVAL;
    if (nb_loc > bte::kMaxBandsPerLaunch)
        return set_err(nullptr, "%d band-rows on one rank (max %d)", nb_loc, bte::kMaxBandsPerLaunch), BTE_EINVAL;

    // --- reflection classes of symmetric faces and their maps (Eq. 6)
    std::map<std::vector<double>, int> cls_of;
    std::vector<int32_t> refl_h;
    std::vector<int32_t> bface_aux(bc->n_bfaces, -1);
    std::vector<double> twall_h;
    for (int64_t c = 0; c < nc64; ++c) {
        for (int64_t f = m->face_offsets[c]; f < m->face_offsets[c + 1]; ++f) {
            if (m->face_nbr[f] >= 0) continue;
            const int64_t bf = -1 - m->face_nbr[f];
            if (bface_aux[bf] >= 0) continue;
            if (bc->kind[bf] == BTE_BC_ISOTHERMAL) {
                bface_aux[bf] = (int32_t)twall_h.size();
                twall_h.push_back(bc->t_wall[bf]);
                continue;
            }
            const double *n = m->face_normal + 3 * f;
            std::vector<double> key(n, n + 3);
            auto it = cls_of.find(key);
            if (it == cls_of.end()) {
                const int id = (int)cls_of.size();
                for (int d = 0; d < nd; ++d) {
                    const double *s = dr->s + 3 * d;
                    const double mu = s[0] * n[0] + s[1] * n[1] + s[2] * n[2];
                    const double r[3] = {s[0] - 2 * mu * n[0], s[1] - 2 * mu * n[1], s[2] - 2 * mu * n[2]};
                    int best = -1;
                    double bestd = 1e300;
                    for (int e = 0; e < nd; ++e) {
                        const double *t = dr->s + 3 * e;
                        const double dd = std::max({std::fabs(t[0] - r[0]), std::fabs(t[1] - r[1]), std::fabs(t[2] - r[2])});
                        if (dd < bestd) bestd = dd, best = e;
                    }
                    if (bestd > 1e-10) {
                        return set_err(nullptr,
                                       "symmetric wall normal (%g,%g,%g): reflection of direction %d is not in the set",
                                       n[0], n[1], n[2], d),
                               BTE_EINVAL;
                    }
                    refl_h.push_back(best);
                }
                it = cls_of.emplace(key, id).first;
            }
            bface_aux[bf] = it->second;
        }
    }

    // --- interior-first cell order
    std::vector<char> is_bnd(nc, 0);
    int mf = 0;
    for (int32_t c = 0; c < nc; ++c) {
        mf = std::max<int>(mf, (int)(m->face_offsets[c + 1] - m->face_offsets[c]));
        for (int64_t f = m->face_offsets[c]; f < m->face_offsets[c + 1]; ++f)
            if (m->face_nbr[f] < 0) is_bnd[c] = 1;
    }
    std::vector<int32_t> user_of, pos_h(nc);
    user_of.reserve(nc);
    for (int32_t c = 0; c < nc; ++c)
        if (!is_bnd[c]) user_of.push_back(c);
    const int32_t n_int = (int32_t)user_of.size();
    for (int32_t c = 0; c < nc; ++c)
        if (is_bnd[c]) user_of.push_back(c);
    for (int32_t i = 0; i < nc; ++i) pos_h[user_of[i]] = i;

    const int mf_t = m->dim == 2 ? (mf <= 4 ? 4 : 8) : (mf <= 6 ? 6 : 8);
    const size_t ell = (size_t)mf_t * nc;
    std::vector<int32_t> nbr_h(ell), aux_h(ell, 0);
    std::vector<double> gx_h(ell, 0.0), gy_h(ell, 0.0), gz_h(ell, 0.0);
    std::vector<int8_t> kind_h(ell, bte::kFaceInterior);
    for (int32_t i = 0; i < nc; ++i) {
        const int32_t c = user_of[i];
        int j = 0;
        for (int64_t f = m->face_offsets[c]; f < m->face_offsets[c + 1]; ++f, ++j) {
            const size_t q = (size_t)j * nc + i;
            const double av = m->face_area[f] / m->cell_volume[c];
            gx_h[q] = av * m->face_normal[3 * f + 0];
            gy_h[q] = av * m->face_normal[3 * f + 1];
            gz_h[q] = av * m->face_normal[3 * f + 2];
            const int64_t nbv = m->face_nbr[f];
            if (nbv >= 0) {
                nbr_h[q] = pos_h[nbv];
            } else {
                const int64_t bf = -1 - nbv;
                nbr_h[q] = i;
                kind_h[q] = bc->kind[bf] == BTE_BC_ISOTHERMAL ? bte::kFaceIso : bte::kFaceSym;
                aux_h[q] = bface_aux[bf];
            }
        }
        for (; j < mf_t; ++j) nbr_h[(size_t)j * nc + i] = i;  // padding: zero geometry
    }

    // --- context
    bte_ctx *ctx = new bte_ctx();
    ctx->opt = *o;
    ctx->dim = m->dim;
    ctx->nd = nd;
    ctx->nb = nb;
    ctx->b_lo = b_lo;
    ctx->b_hi = b_hi;
    ctx->nb_loc = nb_loc;
    ctx->mf = mf;
    ctx->mf_t = mf_t;
    ctx->nc = nc;
    ctx->n_int = n_int;
    ctx->device = o->device;
    ctx->n_iso = (int32_t)twall_h.size();
    ctx->n_refl = (int32_t)cls_of.size();
    ctx->W = 0.0;
    for (int d = 0; d < nd; ++d) ctx->W += dr->w[d];
    auto fail = [&](bte_status s) {
        g_err = ctx->err;
        bte_destroy(ctx);
        return s;
    };
#define CREATE_TRY(call)                    \
    do {                                    \
        bte_status s__ = (call);            \
        if (s__ != BTE_OK) return fail(s__); \
    } while (0)
#define CREATE_CUDA(call)                                                                      \
    do {                                                                                       \
        cudaError_t e_ = (call);                                                               \
        if (e_ != cudaSuccess) {                                                               \
            set_err(&ctx->err, "CUDA error %s at %s:%d", cudaGetErrorString(e_), __FILE__, __LINE__); \
            return fail(e_ == cudaErrorMemoryAllocation ? BTE_ENOMEM : BTE_ECUDA);              \
        }                                                                                      \
    } while (0)

    CREATE_CUDA(cudaSetDevice(o->device));
    {
        cudaDeviceProp prop;
        CREATE_CUDA(cudaGetDeviceProperties(&prop, o->device));
        ctx->sm_count = prop.multiProcessorCount;
        if (prop.major < 10) {
            set_err(&ctx->err, "device %d is sm_%d%d; this library is built for sm_100a", o->device, prop.major, prop.minor);
            return fail(BTE_ECUDA);
        }
    }
    if (o->stream) {
        ctx->stream = (cudaStream_t)o->stream;
    } else {
        CREATE_CUDA(cudaStreamCreateWithFlags(&ctx->stream, cudaStreamNonBlocking));
        ctx->own_stream = true;
    }
    if (o->world > 1 && o->nccl_unique_id) {
        std::string e;
        if (!bte::nccl::init(&ctx->comm, o->nccl_unique_id, o->rank, o->world, &e)) {
            set_err(&ctx->err, "NCCL init failed: %s", e.c_str());
            return fail(BTE_ENCCL);
        }
        ctx->have_comm = true;
    }

    // --- launch plan knobs
    ctx->block = o->block_threads > 0 ? std::max(32, std::min(bte::kMaxThreads, o->block_threads / 32 * 32)) : 256;
    ctx->bg = round_bg(o->band_group > 0 ? o->band_group : 4);

    // --- slab pool: nb_loc current slabs + n_spare workspace slabs
    ctx->slab_elems = (int64_t)nd * nc;
    const size_t slab_bytes = (size_t)ctx->slab_elems * sizeof(double);
    int n_spare = nb_loc;
    if (o->max_spare_slabs > 0) n_spare = std::min(n_spare, (int)o->max_spare_slabs);
    {
        size_t free_b = 0, total_b = 0;
        CREATE_CUDA(cudaMemGetInfo(&free_b, &total_b));
        const size_t other = (size_t)nc * sizeof(double) * (size_t)(3 * nb_loc + 16) + ell * 40 + (64u << 20);
        const size_t reserve = (size_t)1 << 30;
        while (n_spare > 1 && (size_t)(nb_loc + n_spare) * slab_bytes + other + reserve > free_b) --n_spare;
        if ((size_t)(nb_loc + n_spare) * slab_bytes + other > free_b) {
            set_err(&ctx->err, "intensity needs %.1f GB (%d slabs of %.2f GB); %.1f GB free",
                    (nb_loc + n_spare) * slab_bytes / 1e9, nb_loc + n_spare, slab_bytes / 1e9, free_b / 1e9);
            return fail(BTE_ENOMEM);
        }
    }
    ctx->n_spare = n_spare;
    ctx->bg = std::min(ctx->bg, round_bg(n_spare));
    while (ctx->bg > n_spare) ctx->bg /= 2;
    ctx->cur_slot.resize(nb_loc);
    ctx->spare_slot.resize(n_spare);
    for (int k = 0; k < nb_loc; ++k) ctx->cur_slot[k] = k;
    for (int k = 0; k < n_spare; ++k) ctx->spare_slot[k] = nb_loc + k;
    CREATE_TRY(dalloc(ctx, &ctx->pool, (size_t)(nb_loc + n_spare) * ctx->slab_elems));

    // --- energy partial slots: worst case over the launch batches
    int max_slots = 0;
    for (int l0 = 0; l0 < nb_loc; l0 += n_spare) {
        const int nbl = std::min(n_spare, nb_loc - l0);
        LaunchPlan lp = plan_launch(ctx, nbl, n_int > 0 ? n_int : nc - n_int);
        max_slots += lp.groups * lp.n_dch;
    }
    CREATE_TRY(dalloc(ctx, &ctx->part, (size_t)max_slots * nc));
    CREATE_TRY(dalloc(ctx, &ctx->i0, (size_t)nb_loc * nc));
    CREATE_TRY(dalloc(ctx, &ctx->T, (size_t)nc));
    CREATE_TRY(dalloc(ctx, &ctx->E, (size_t)nc));
    ctx->staging_elems = std::min<int64_t>(ctx->slab_elems, std::max<int64_t>(nc, (int64_t)8 << 20));
    CREATE_TRY(dalloc(ctx, &ctx->staging, (size_t)ctx->staging_elems));
    CREATE_TRY(upload(ctx, &ctx->d_cur_slot, ctx->cur_slot));
    CREATE_TRY(upload(ctx, &ctx->nbr, nbr_h));
    CREATE_TRY(upload(ctx, &ctx->aux, aux_h));
    CREATE_TRY(upload(ctx, &ctx->kind, kind_h));
    CREATE_TRY(upload(ctx, &ctx->gx, gx_h));
    CREATE_TRY(upload(ctx, &ctx->gy, gy_h));
    CREATE_TRY(upload(ctx, &ctx->gz, gz_h));
    CREATE_TRY(upload(ctx, &ctx->pos, pos_h));
    CREATE_TRY(upload(ctx, &ctx->refl, refl_h));
    CREATE_TRY(upload(ctx, &ctx->twall, twall_h));
    std::vector<double4> dirs_h(nd);
    for (int d = 0; d < nd; ++d) dirs_h[d] = make_double4(dr->s[3 * d], dr->s[3 * d + 1], dr->s[3 * d + 2], dr->w[d]);
    CREATE_TRY(upload(ctx, &ctx->dirs, dirs_h));
    std::vector<double> it_loc(inv_tau.begin() + b_lo, inv_tau.begin() + b_hi);
    std::vector<double> vg_loc(bd->vg + b_lo, bd->vg + b_hi);
    std::vector<double> cw_loc(cw.begin() + b_lo, cw.begin() + b_hi);
    CREATE_TRY(upload(ctx, &ctx->inv_tau, it_loc));
    CREATE_TRY(upload(ctx, &ctx->vg, vg_loc));
    CREATE_TRY(upload(ctx, &ctx->cw_loc, cw_loc));
    CREATE_TRY(upload(ctx, &ctx->Cb, std::vector<double>(bd->i0_prefactor, bd->i0_prefactor + nb)));
    CREATE_TRY(upload(ctx, &ctx->theta, theta));
    CREATE_TRY(upload(ctx, &ctx->cw_all, cw));
    CREATE_TRY(dalloc(ctx, &ctx->i0w, (size_t)nb_loc * std::max(1, ctx->n_iso)));
    CREATE_TRY(dalloc(ctx, &ctx->d_iter_max, 1));
    CREATE_TRY(dalloc(ctx, &ctx->d_fail, 1));
    CREATE_TRY(dalloc(ctx, &ctx->d_smax, 1));
    CREATE_CUDA(cudaMemsetAsync(ctx->d_iter_max, 0, sizeof(int32_t), ctx->stream));
    CREATE_CUDA(cudaMemsetAsync(ctx->d_fail, 0, sizeof(int32_t), ctx->stream));
    CREATE_CUDA(cudaMemsetAsync(ctx->d_smax, 0, sizeof(unsigned long long), ctx->stream));

    // --- initial state: T = t_init, I = I0_b(t_init); ghost table; dt bound
    {
        std::vector<double> T0(nc, o->t_init);
        CREATE_CUDA(cudaMemcpy(ctx->T, T0.data(), nc * sizeof(double), cudaMemcpyHostToDevice));
        const int tb = 256;
        const int gb = (nc + tb - 1) / tb;
        bte::i0_table_kernel<<<gb, tb, 0, ctx->stream>>>(ctx->T, nc, b_lo, nb_loc, ctx->Cb, ctx->theta, ctx->i0);
        bte::equilibrium_kernel<<<dim3(std::min<int64_t>(4096, (ctx->slab_elems + tb - 1) / tb), nb_loc), tb, 0,
                                  ctx->stream>>>(ctx->pool, ctx->d_cur_slot, ctx->slab_elems, nd, nc, ctx->i0);
        if (ctx->n_iso > 0)
            bte::i0w_kernel<<<(ctx->n_iso + tb - 1) / tb, tb, 0, ctx->stream>>>(ctx->twall, ctx->n_iso, b_lo, nb_loc,
                                                                               ctx->Cb, ctx->theta, ctx->i0w);
        if (m->dim == 2)
            bte::outflow_max_kernel<2><<<gb, tb, 0, ctx->stream>>>(nc, mf_t, nd, ctx->gx, ctx->gy, ctx->gz, ctx->dirs, ctx->d_smax);
        else
            bte::outflow_max_kernel<3><<<gb, tb, 0, ctx->stream>>>(nc, mf_t, nd, ctx->gx, ctx->gy, ctx->gz, ctx->dirs, ctx->d_smax);
        CREATE_CUDA(cudaGetLastError());
        unsigned long long bits = 0;
        CREATE_CUDA(cudaMemcpyAsync(&bits, ctx->d_smax, sizeof bits, cudaMemcpyDeviceToHost, ctx->stream));
        CREATE_CUDA(cudaStreamSynchronize(ctx->stream));
        std::memcpy(&ctx->s_max, &bits, sizeof(double));
        double rate = 0.0;
        for (int b = 0; b < nb; ++b) rate = std::max(rate, inv_tau[b] + bd->vg[b] * ctx->s_max);
        ctx->dt_bound = rate > 0.0 ? 1.0 / rate : INFINITY;
    }
    ctx->st.spare_slabs = n_spare;
    ctx->st.n_interior_cells = n_int;
    ctx->st.band_group = ctx->bg;
    ctx->st.block_threads = ctx->block;
    *out = ctx;
    return BTE_OK;
#undef CREATE_TRY
#undef CREATE_CUDA
}

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

static bte_status check_dt(bte_ctx *ctx, double dt) {
    if (!(dt > 0.0) || !std::isfinite(dt)) return set_err(&ctx->err, "dt must be > 0 (got %g)", dt), BTE_EINVAL;
    if (dt > ctx->dt_bound * (1.0 + 1e-12))
        return set_err(&ctx->err, "dt = %.6g exceeds the positivity bound %.6g", dt, ctx->dt_bound), BTE_EINVAL;
    return BTE_OK;
}

bte_status bte_step(bte_ctx *ctx, double dt, int64_t n) {
    if (!ctx) return BTE_EINVAL;
    if (ctx->begun) return set_err(&ctx->err, "split step in flight"), BTE_ESTATE;
    if (n < 0) return set_err(&ctx->err, "n < 0"), BTE_EINVAL;
    if (n == 0) return BTE_OK;
    STATUS_TRY(check_dt(ctx, dt));
    if (ctx->opt.world > 1 && !ctx->have_comm)
        return set_err(&ctx->err, "world > 1 without a communicator: reduce the energy with "
                                  "bte_step_begin / bte_get_energy / bte_set_energy / bte_step_finish"), BTE_ESTATE;
    CUDA_TRY(ctx, cudaSetDevice(ctx->device));
    for (int64_t s = 0; s < n; ++s) {
        STATUS_TRY(run_flux(ctx, dt));
        if (ctx->opt.world > 1) {
            ev_mark(ctx, kPhAllreduce, true);
            STATUS_TRY(reduce_slots(ctx));
            STATUS_TRY(allreduce_E(ctx));
            ev_mark(ctx, kPhAllreduce, false);
            STATUS_TRY(run_newton(ctx, ctx->E));
        } else {
            STATUS_TRY(run_newton(ctx, nullptr));
        }
        ctx->st.steps++;
        ctx->st.updates += (int64_t)ctx->nc * ctx->nd * ctx->nb_loc;
    }
    STATUS_TRY(upload_cur_slots(ctx));
    return check_newton(ctx);
}

bte_status bte_step_begin(bte_ctx *ctx, double dt) {
    if (!ctx) return BTE_EINVAL;
    if (ctx->begun) return set_err(&ctx->err, "split step already begun"), BTE_ESTATE;
    STATUS_TRY(check_dt(ctx, dt));
    CUDA_TRY(ctx, cudaSetDevice(ctx->device));
    STATUS_TRY(run_flux(ctx, dt));
    STATUS_TRY(reduce_slots(ctx));
    STATUS_TRY(upload_cur_slots(ctx));
    CUDA_TRY(ctx, cudaStreamSynchronize(ctx->stream));
    ctx->begun = true;
    ctx->begun_dt = dt;
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

// rows of nc doubles between a device array (internal order) and a host array (caller order)
static bte_status rows_to_host(const bte_ctx *cctx, const double *dsrc, int64_t rows, double *host) {
    bte_ctx *ctx = const_cast<bte_ctx *>(cctx);
    const int64_t per = std::max<int64_t>(1, ctx->staging_elems / ctx->nc);
    for (int64_t r0 = 0; r0 < rows; r0 += per) {
        const int64_t nr = std::min(per, rows - r0);
        const int64_t n = nr * ctx->nc;
        const int tb = 256;
        const int gb = (int)std::min<int64_t>(8192, (n + tb - 1) / tb);
        bte::gather_rows_kernel<<<gb, tb, 0, ctx->stream>>>(dsrc + r0 * ctx->nc, ctx->pos, ctx->nc, nr, ctx->staging);
        CUDA_TRY(ctx, cudaGetLastError());
        CUDA_TRY(ctx, cudaMemcpyAsync(host + r0 * ctx->nc, ctx->staging, n * sizeof(double), cudaMemcpyDeviceToHost,
                                      ctx->stream));
        CUDA_TRY(ctx, cudaStreamSynchronize(ctx->stream));
    }
    return BTE_OK;
}

static bte_status rows_from_host(bte_ctx *ctx, const double *host, int64_t rows, double *ddst) {
    const int64_t per = std::max<int64_t>(1, ctx->staging_elems / ctx->nc);
    for (int64_t r0 = 0; r0 < rows; r0 += per) {
        const int64_t nr = std::min(per, rows - r0);
        const int64_t n = nr * ctx->nc;
        CUDA_TRY(ctx, cudaMemcpyAsync(ctx->staging, host + r0 * ctx->nc, n * sizeof(double), cudaMemcpyHostToDevice,
                                      ctx->stream));
        const int tb = 256;
        const int gb = (int)std::min<int64_t>(8192, (n + tb - 1) / tb);
        bte::scatter_rows_kernel<<<gb, tb, 0, ctx->stream>>>(ctx->staging, ctx->pos, ctx->nc, nr, ddst + r0 * ctx->nc);
        CUDA_TRY(ctx, cudaGetLastError());
        CUDA_TRY(ctx, cudaStreamSynchronize(ctx->stream));
    }
    return BTE_OK;
}

bte_status bte_get_temperature(const bte_ctx *ctx, double *T) {
    if (!ctx || !T) return BTE_EINVAL;
    CUDA_TRY(const_cast<bte_ctx *>(ctx), cudaSetDevice(ctx->device));
    return rows_to_host(ctx, ctx->T, 1, T);
}

bte_status bte_get_energy(const bte_ctx *ctx, double *E) {
    if (!ctx || !E) return BTE_EINVAL;
    CUDA_TRY(const_cast<bte_ctx *>(ctx), cudaSetDevice(ctx->device));
    return rows_to_host(ctx, ctx->E, 1, E);
}

bte_status bte_set_energy(bte_ctx *ctx, const double *E) {
    if (!ctx || !E) return BTE_EINVAL;
    CUDA_TRY(ctx, cudaSetDevice(ctx->device));
    return rows_from_host(ctx, E, 1, ctx->E);
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
        const double *slab = ctx->pool + (int64_t)ctx->cur_slot[b - ctx->b_lo] * ctx->slab_elems;
        STATUS_TRY(rows_to_host(ctx, slab, ctx->nd, I + (int64_t)(b - b_lo) * ctx->slab_elems));
    }
    return BTE_OK;
}

bte_status bte_set_intensity(bte_ctx *ctx, int32_t b_lo, int32_t b_hi, const double *I) {
    if (!ctx || !I) return BTE_EINVAL;
    STATUS_TRY(check_rows(ctx, b_lo, b_hi));
    CUDA_TRY(ctx, cudaSetDevice(ctx->device));
    for (int32_t b = b_lo; b < b_hi; ++b) {
        double *slab = ctx->pool + (int64_t)ctx->cur_slot[b - ctx->b_lo] * ctx->slab_elems;
        STATUS_TRY(rows_from_host(ctx, I + (int64_t)(b - b_lo) * ctx->slab_elems, ctx->nd, slab));
    }
    return BTE_OK;
}

bte_status bte_solve_temperature(bte_ctx *ctx) {
    if (!ctx) return BTE_EINVAL;
    if (ctx->begun) return BTE_ESTATE;
    if (ctx->opt.world > 1 && !ctx->have_comm)
        return set_err(&ctx->err, "world > 1 without a communicator: cannot reduce the energy"), BTE_ESTATE;
    CUDA_TRY(ctx, cudaSetDevice(ctx->device));
    const int tb = 128;
    bte::energy_kernel<<<(ctx->nc + tb - 1) / tb, tb, 0, ctx->stream>>>(
        ctx->pool, ctx->d_cur_slot, ctx->slab_elems, ctx->nb_loc, ctx->nd, ctx->nc, ctx->dirs, ctx->cw_loc, ctx->E);
    CUDA_TRY(ctx, cudaGetLastError());
    STATUS_TRY(allreduce_E(ctx));
    STATUS_TRY(run_newton(ctx, ctx->E));
    return check_newton(ctx);
}

bte_status bte_set_equilibrium(bte_ctx *ctx, const double *T) {
    if (!ctx || !T) return BTE_EINVAL;
    if (ctx->begun) return BTE_ESTATE;
    CUDA_TRY(ctx, cudaSetDevice(ctx->device));
    for (int32_t c = 0; c < ctx->nc; ++c)
        if (!(T[c] > 0.0) || !std::isfinite(T[c])) return set_err(&ctx->err, "T[%d] must be > 0", c), BTE_EINVAL;
    STATUS_TRY(rows_from_host(ctx, T, 1, ctx->T));
    STATUS_TRY(refresh_i0(ctx));
    const int tb = 256;
    bte::equilibrium_kernel<<<dim3(std::min<int64_t>(4096, (ctx->slab_elems + tb - 1) / tb), ctx->nb_loc), tb, 0,
                              ctx->stream>>>(ctx->pool, ctx->d_cur_slot, ctx->slab_elems, ctx->nd, ctx->nc, ctx->i0);
    CUDA_TRY(ctx, cudaGetLastError());
    CUDA_TRY(ctx, cudaStreamSynchronize(ctx->stream));
    return BTE_OK;
}

bte_status bte_get_stats(const bte_ctx *ctx, bte_stats *st) {
    if (!ctx || !st) return BTE_EINVAL;
    *st = ctx->st;
    st->dir_chunks = ctx->dir_chunks;
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
    return BTE_OK;
}

}  // extern "C"
