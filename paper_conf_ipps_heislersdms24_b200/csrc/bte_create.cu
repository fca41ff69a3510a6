// bte_create.cu -- bte_create / bte_destroy (see bte_internal.h): validation
// of the problem statement, detection of the structured grids the box kernel
// takes (2-D / 3-D boxes, z-slab cell partitions), the cell order, face slots,
// reflection maps, isothermal tables, slab pool, tensor maps and the
// equilibrium initial state.
#include "bte_internal.h"
#include "bte_staging.h"
#include <map>
#include <set>
#include <cstring>

namespace bte_host {


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

// ------------------------------------------------------------- built-in dispersion
// I0 prefactor C_b when the caller passes none (bte_bands.i0_prefactor NULL):
// the intensity of a band of width d_omega at its centre frequency omega is
// I0_b(T) = C_b / expm1(hbar omega / (kB T)) with C_b = hbar omega k^2 d_omega / (8 pi^3)
// (I = v_g hbar omega f D(omega) / (4 pi), D = k^2 / (2 pi^2 v_g)),
// k from the quadratic Si dispersion omega = v_s k + c k^2 of the row's branch
// (LA v_s = 9.01e3 m/s, c = -2.0e-7 m^2/s; TA 5.23e3, -2.26e-7),
// the stable root k = 2 omega / (v_s + sqrt(v_s^2 + 4 c omega)).  External
// physics (the paper defers the relation to [14], [4], L559-561).
bte_status derive_prefactors(const bte_bands *b, std::vector<double> *C) {
    static const double vs[2] = {9.01e3, 5.23e3}, cq[2] = {-2.0e-7, -2.26e-7};
    C->resize(b->n_bands);
    for (int i = 0; i < b->n_bands; ++i) {
        if (b->i0_prefactor) {
            (*C)[i] = b->i0_prefactor[i];
            continue;
        }
        const int pol = b->polarization[i];
        if (pol != 0 && pol != 1) return set_err(nullptr, "band-row %d: polarization must be 0 (LA) or 1 (TA)", i), BTE_EINVAL;
        const double w = b->omega[i], disc = vs[pol] * vs[pol] + 4.0 * cq[pol] * w;
        if (!(disc > 0.0))
            return set_err(nullptr, "band-row %d: omega %g above the built-in dispersion's branch maximum", i, w),
                   BTE_EINVAL;
        const double k = 2.0 * w / (vs[pol] + std::sqrt(disc));
        (*C)[i] = kHbar * w * k * k * b->d_omega[i] / (8.0 * std::pow(M_PI, 3));
    }
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
    if (m->n_cells <= 0 || m->n_cells >= (int64_t)1 << 30)
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
    std::vector<char> seen(bc->n_bfaces > 0 ? bc->n_bfaces : 0, 0);
    for (int64_t f = 0; f < nfaces; ++f) {
        if (!(m->face_area[f] > 0.0)) return set_err(nullptr, "face %lld area <= 0", (long long)f), BTE_EINVAL;
        const double *n = m->face_normal + 3 * f;
        if (!unit(n, 1e-9)) return set_err(nullptr, "face %lld normal not unit", (long long)f), BTE_EINVAL;
        if (m->dim == 2 && n[2] != 0.0) return set_err(nullptr, "2-D mesh with n_z != 0 (face %lld)", (long long)f), BTE_EINVAL;
        const int64_t nb = m->face_nbr[f];
        if (nb >= m->n_cells) return set_err(nullptr, "face %lld neighbour out of range", (long long)f), BTE_EINVAL;
        if (nb < 0) {
            const int64_t bf = -1 - nb;
            if (bf >= bc->n_bfaces) return set_err(nullptr, "face %lld boundary id out of range", (long long)f), BTE_EINVAL;
            if (seen[bf]++) return set_err(nullptr, "boundary face id %lld used twice", (long long)bf), BTE_EINVAL;
        }
    }
    const bool law = b->rate_a != nullptr;
    if (b->n_bands < 1 || !b->omega || !b->vg || (!b->tau && !law))
        return set_err(nullptr, "band table incomplete"), BTE_EINVAL;
    if (law && (!b->rate_b || !b->rate_theta))
        return set_err(nullptr, "rate law needs rate_a, rate_b and rate_theta"), BTE_EINVAL;
    for (int i = 0; law && i < b->n_bands; ++i)
        if (!(b->rate_a[i] >= 0.0) || !(b->rate_b[i] >= 0.0) || !(b->rate_theta[i] >= 0.0) ||
            !std::isfinite(b->rate_a[i]) || !std::isfinite(b->rate_b[i]) || !std::isfinite(b->rate_theta[i]))
            return set_err(nullptr, "band-row %d: rate law coefficients must be finite and >= 0", i), BTE_EINVAL;
    if (b->n_bands > bte::kMaxBands)
        return set_err(nullptr, "%d band-rows (max %d)", b->n_bands, bte::kMaxBands), BTE_EINVAL;
    if (!b->i0_prefactor && (!b->d_omega || !b->polarization))
        return set_err(nullptr, "i0_prefactor NULL: d_omega and polarization are needed to derive C_b"), BTE_EINVAL;
    for (int i = 0; i < b->n_bands; ++i) {
        if (!(b->omega[i] > 0.0) || !(b->vg[i] > 0.0) || !(law || b->tau[i] > 0.0) ||
            !(b->i0_prefactor ? b->i0_prefactor[i] > 0.0 : b->d_omega[i] > 0.0))
            return set_err(nullptr, "band-row %d: omega, vg, tau, C (or d_omega) must be > 0", i), BTE_EINVAL;
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
    if (o->temp_rule < 0 || o->temp_rule > 2) return set_err(nullptr, "temp_rule must be 0, 1 or 2"), BTE_EINVAL;
    if (!(o->t_init > 0.0)) return set_err(nullptr, "t_init must be > 0"), BTE_EINVAL;
    if (o->world < 1 || o->rank < 0 || o->rank >= o->world) return set_err(nullptr, "bad rank/world"), BTE_EINVAL;
    if (!(o->newton_rtol > 0.0) || o->newton_max_iter < 1) return set_err(nullptr, "bad Newton controls"), BTE_EINVAL;
    if (o->group && (!o->group->g || bte::group::world_of(o->group->g) != o->world))
        return set_err(nullptr, "in-process group of %d ranks with world %d", bte::group::world_of(o->group ? o->group->g : nullptr),
                       o->world), BTE_EINVAL;
    if (o->group && o->nccl_unique_id) return set_err(nullptr, "pass either a group or an NCCL id"), BTE_EINVAL;
    return BTE_OK;
}

}  // namespace bte_host

using namespace bte_host;

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

bte_status bte_group_create(int32_t world, bte_group **out) {
    if (!out || world < 1) return set_err(nullptr, "bte_group_create: world >= 1 and out needed"), BTE_EINVAL;
    *out = new bte_group();
    (*out)->g = bte::group::create(world);
    return BTE_OK;
}

void bte_group_destroy(bte_group *g) {
    if (!g) return;
    bte::group::destroy(g->g);
    delete g;
}

void bte_destroy(bte_ctx *ctx) {
    if (!ctx) return;
    cudaSetDevice(ctx->device);
    if (ctx->stream) cudaStreamSynchronize(ctx->stream);
    if (ctx->gexec) cudaGraphExecDestroy(ctx->gexec);
    if (ctx->own_bcomm) bte::nccl::destroy(ctx->bcomm);
    if (ctx->have_comm) bte::nccl::destroy(ctx->comm);
    for (HaloSeg &h : ctx->hsegs) {
        void *hp[] = {h.send_cells, h.send_dirs, h.recv_dirs, h.recv_cols, h.sbuf, h.rbuf};
        for (void *q : hp)
            if (q) cudaFree(q);
    }
    void *ptrs[] = {ctx->pool, ctx->d_cur_slot, ctx->i0, ctx->T, ctx->E,
                    ctx->part, ctx->staging, ctx->nbr, ctx->nbm, ctx->fcode, ctx->fcode8, ctx->pos, ctx->gx,
                    ctx->gy, ctx->gz, ctx->refl, ctx->i0w, ctx->twall, ctx->dirs, ctx->cw_loc, ctx->Cb, ctx->theta, ctx->cw_all,
                    ctx->d_iter_max, ctx->d_flags, ctx->d_smax, ctx->t_th, ctx->t_k, ctx->t_ic, ctx->t_rep, ctx->orb, ctx->dirs_box, ctx->side_tab, ctx->side_col,
                    ctx->d_ra, ctx->d_rb, ctx->d_rth, ctx->d_inv_v, ctx->rates, ctx->Tr,
                    ctx->E2, ctx->T2, ctx->cw_diag, ctx->Echunk, ctx->Tg, ctx->hl_off, ctx->hl_cell, ctx->hl_pos, ctx->sidx, ctx->bl_off, ctx->bl_col, ctx->bl_cls, ctx->bl_pos,
                    ctx->t_nrow, ctx->fresh};
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
    std::vector<double> Cb_all;  // I0 prefactors (given, or from the built-in dispersion)
    STATUS_TRY(derive_prefactors(bd, &Cb_all));
    // --- cell partitioning (N3): rank r owns part r % P of the cells and band
    // group r / P; from here on `m` is the owned cells' mesh with halo columns
    const bool cpart = o->cell_part != nullptr;
    const int n_parts = cpart ? o->n_cell_parts : 1;
    if (cpart && (n_parts < 1 || o->world % n_parts != 0))
        return set_err(nullptr, "world %d is not a multiple of n_cell_parts %d", o->world, n_parts), BTE_EINVAL;
    const int my_part = o->rank % n_parts, G = o->world / n_parts, gband = o->rank / n_parts;
    LocalPlan lplan;
    ZSlab zs;
    if (cpart) {
        zs = detect_zslab(m, dr, bc, o, my_part);
        STATUS_TRY(build_local(m, dr, o, my_part, &lplan));
        m = &lplan.mesh;
    }
    const int32_t n_halo = lplan.n_halo;
    const int nd = dr->n_dirs, nb = bd->n_bands;
    const int64_t nc64 = m->n_cells;
    const int32_t nc = (int32_t)nc64;

    // --- temperature weights c_b and band constants
    std::vector<double> cw(nb), theta(nb), inv_tau(nb);
    bool any_w = false;
    const bool td = bd->rate_a != nullptr;  // rate law (N1): the constants below at t_init
    for (int b = 0; b < nb; ++b) {
        if (td) inv_tau[b] = bd->rate_a[b] + bd->rate_b[b] * o->t_init * std::exp(-bd->rate_theta[b] / o->t_init);
        else inv_tau[b] = std::isinf(bd->tau[b]) ? 0.0 : 1.0 / bd->tau[b];
        cw[b] = o->temp_rule != 0 ? 1.0 / bd->vg[b] : inv_tau[b] / bd->vg[b];  // R1 / R3: 1/v_b
        if (!td && o->temp_rule == 0) cw[b] = std::isinf(bd->tau[b]) ? 0.0 : 1.0 / (bd->vg[b] * bd->tau[b]);
        theta[b] = kHbar * bd->omega[b] / kKb;
        any_w |= cw[b] > 0.0 || (td && o->temp_rule == 0 && bd->rate_b[b] > 0.0);
    }
    if (!any_w) return set_err(nullptr, "all temperature weights are zero (temp_rule 0 with every tau = inf)"), BTE_EINVAL;

    // --- band sharding: rank g owns [floor(g nb/P), floor((g+1) nb/P))  (L760-775)
    const int b_lo = (int)((int64_t)gband * nb / G);
    const int b_hi = (int)((int64_t)(gband + 1) * nb / G);
    const int nb_loc = b_hi - b_lo;
    if (nb_loc < 1) return set_err(nullptr, "rank %d owns no band-row (n_bands %d < band groups %d)", o->rank, nb, G), BTE_EINVAL;
    if (nb_loc > bte::kMaxBandsPerLaunch)
        return set_err(nullptr, "%d band-rows on one rank (max %d)", nb_loc, bte::kMaxBandsPerLaunch), BTE_EINVAL;

    // --- face pairing: every face of every cell has an exactly opposite partner
    // (same area, negated normal) -> paired layout, one upwind load per pair.
    int mf = 0;
    for (int64_t c = 0; c < nc64; ++c) mf = std::max<int>(mf, (int)(m->face_offsets[c + 1] - m->face_offsets[c]));
    std::vector<int64_t> partner(m->face_offsets[nc64], -1);
    bool paired_geom = mf <= 2 * m->dim && !(o->flags & BTE_FLAG_GENERIC_FACES);
    for (int64_t c = 0; c < nc64 && paired_geom; ++c) {
        const int64_t f0 = m->face_offsets[c], f1 = m->face_offsets[c + 1];
        for (int64_t f = f0; f < f1 && paired_geom; ++f) {
            if (partner[f] >= 0) continue;
            const double *n = m->face_normal + 3 * f;
            for (int64_t g = f + 1; g < f1; ++g) {
                const double *q = m->face_normal + 3 * g;
                if (partner[g] < 0 && m->face_area[g] == m->face_area[f] && q[0] == -n[0] && q[1] == -n[1] &&
                    q[2] == -n[2]) {
                    partner[f] = g;
                    partner[g] = f;
                    break;
                }
            }
            if (partner[f] < 0) paired_geom = false;
        }
    }
    // --- structured box grid -> the box kernel (grid lexicographic order)
    BoxDetect bx;
    std::vector<bte::BoxOrbit> orbs;
    if (paired_geom && !cpart && !(o->flags & (BTE_FLAG_NO_BOX | BTE_FLAG_NO_TMA)))
        bx = m->dim == 3 ? detect_box(m, bc) : detect_box2d(m, bc);
    if (zs.on) {  // z-slab partition: the owned layers of the global box, in grid order (local ids)
        const BoxDetect &g = zs.gbx;
        const int64_t plane = (int64_t)g.n[0] * g.n[1];
        bx = g;
        bx.n[2] = zs.zb - zs.za;
        for (int sd = 0; sd < 2; ++sd)  // a side facing a neighbour part reads its halo layer, never a wall
            if (sd ? zs.h_hi : zs.h_lo) bx.zside[sd] = 1;
        bx.cell_at.resize((size_t)plane * bx.n[2]);
        for (int64_t i = 0; i < (int64_t)bx.cell_at.size(); ++i) {
            const int64_t gcell = g.cell_at[(int64_t)zs.za * plane + i];
            bx.cell_at[i] = (int32_t)(std::lower_bound(lplan.gid.begin(), lplan.gid.end(), gcell) - lplan.gid.begin());
        }
        orbs = zs.orbs;
    }
    // (the box kernel addresses a slab with 32-bit plane offsets: nd x padded cells < 2^31)
    const bool box_fits = (int64_t)nd * ((nc64 + n_halo + bte::kTile - 1) / bte::kTile * bte::kTile) < INT32_MAX;
    const bool use_box = bx.ok && box_fits && (zs.on || box_orbits(dr, bx.ax, !bx.flat && (bx.zside[0] == 1 || bx.zside[1] == 1), &orbs));

    // --- internal cell order from the optional centroids: cells are grouped
    // into bricks of 8 x 8 x 4 (2-D: 16 x 16) typical cell sizes, Morton order
    // inside a brick (a 256-cell thread block is one brick), bricks in
    // row-major order with the axis of most bricks slowest, so every face
    // neighbour of a brick is at most (bricks per slab) blocks away and its
    // upwind data is still in L2 when needed.  Else: the caller's order.
    // pos_h: caller -> internal.
    std::vector<int32_t> user_of(nc), pos_h(nc);
    for (int32_t c = 0; c < nc; ++c) user_of[c] = c;
    const bool use_locality = !use_box && m->cell_centre;
    if (use_box) {
        user_of = bx.cell_at;
    } else if (use_locality) {
        const int D = m->dim;
        double lo[3] = {INFINITY, INFINITY, INFINITY}, hi[3] = {-INFINITY, -INFINITY, -INFINITY};
        for (int32_t c = 0; c < nc; ++c)
            for (int a = 0; a < D; ++a) {
                lo[a] = std::min(lo[a], m->cell_centre[3 * c + a]);
                hi[a] = std::max(hi[a], m->cell_centre[3 * c + a]);
            }
        double vol = 1.0;
        for (int a = 0; a < D; ++a) vol *= std::max(hi[a] - lo[a], 1e-300);
        const double h = std::pow(vol / (double)nc, 1.0 / D);  // typical cell size
        const double bsz[3] = {8.0 * h, 8.0 * h, (D == 3 ? 4.0 : 16.0) * h};
        const double bsz2[3] = {16.0 * h, 16.0 * h, 1.0};
        const double *B = D == 3 ? bsz : bsz2;
        int64_t nbk[3] = {1, 1, 1};
        for (int a = 0; a < D; ++a) nbk[a] = (int64_t)std::floor((hi[a] - lo[a]) / B[a]) + 1;
        int ax[3] = {0, 1, 2};  // brick axes, slowest first: the axis with the most bricks
        std::sort(ax, ax + D, [&](int a, int b) { return nbk[a] > nbk[b]; });
        std::vector<uint64_t> key(nc);
        for (int32_t c = 0; c < nc; ++c) {
            uint64_t bidx = 0, loc[3] = {0, 0, 0};
            for (int t = 0; t < D; ++t) {
                const int a = ax[t];
                const double r = (m->cell_centre[3 * c + a] - lo[a]) / B[a];
                const int64_t bi = std::min<int64_t>(nbk[a] - 1, std::max<int64_t>(0, (int64_t)std::floor(r)));
                bidx = bidx * (uint64_t)nbk[a] + (uint64_t)bi;
                loc[a] = (uint64_t)std::min(1023.0, std::max(0.0, std::floor((r - bi) * 1024.0)));
            }
            uint64_t mort = 0;  // Morton code of the position inside the brick (10 bits per axis)
            for (int bit = 9; bit >= 0; --bit)
                for (int a = 0; a < D; ++a) mort = (mort << 1) | ((loc[a] >> bit) & 1u);
            key[c] = (bidx << 30) | mort;
        }
        std::stable_sort(user_of.begin(), user_of.end(), [&](int32_t a, int32_t b) { return key[a] < key[b]; });
    }
    for (int32_t i = 0; i < nc; ++i) pos_h[user_of[i]] = i;

    // --- boundary faces: isothermal table columns (internal cell order) and
    // reflection classes of specular faces with their maps (Eq. 6)
    std::map<std::vector<double>, int> cls_of;
    std::vector<int32_t> refl_h, iso_of(bc->n_bfaces, -1), bcls(bc->n_bfaces, -1);
    std::vector<double> twall_h;
    int32_t n_bcells = 0;
    for (int32_t i = 0; i < nc; ++i) {
        const int64_t c = user_of[i];
        bool bcell = false;
        for (int64_t f = m->face_offsets[c]; f < m->face_offsets[c + 1]; ++f) {
            if (m->face_nbr[f] >= 0) continue;
            bcell = true;
            const int64_t bf = -1 - m->face_nbr[f];
            if (bc->kind[bf] == BTE_BC_ISOTHERMAL) {
                iso_of[bf] = (int32_t)twall_h.size();
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
            bcls[bf] = it->second;
        }
        n_bcells += bcell;
    }

    if ((int)cls_of.size() > bte::kMaxGenericClasses)
        return set_err(nullptr, "%d distinct specular wall normals (max %d)", (int)cls_of.size(),
                       bte::kMaxGenericClasses), BTE_EINVAL;

    // --- plane stride: cells (and halo columns) padded to a whole 256-cell tile (2 KB)
    const int32_t ps = (int32_t)((nc64 + n_halo + bte::kTile - 1) / bte::kTile * bte::kTile);

    // (the paired layout's 5-bit face codes hold up to 16 specular classes)
    // (with the rate law only the box kernel and the generic-face kernel read rate tables)
    // (the opposite-pair layout feeds the TMA-staged paired kernel only: 256-thread blocks)
    const int32_t block = o->block_threads > 0 ? std::max(32, std::min(bte::kMaxThreads, o->block_threads / 32 * 32)) : 256;
    const bool tma_ok = block == bte::kTile && !(o->flags & BTE_FLAG_NO_TMA);
    const bool paired = paired_geom && tma_ok && (int)cls_of.size() <= bte::kMaxPairedClasses && !(td && !use_box);
    const int mf_t = paired ? m->dim
                            : (m->dim == 2 ? (mf <= 3 ? 3 : mf <= 4 ? 4 : 8) : (mf <= 4 ? 4 : mf <= 6 ? 6 : 8));
    const size_t ell = (size_t)mf_t * nc;
    std::vector<int32_t> nbr_h(ell), nbm_h(paired ? ell : 1, 0);
    std::vector<uint32_t> fcode_h(paired ? nc : 1, (1u << (10 * m->dim)) - 1u);  // all interior
    std::vector<uint8_t> fcode8_h(paired ? 1 : ell, (uint8_t)bte::kCode8Interior);
    std::vector<double> gx_h(ell, 0.0), gy_h(ell, 0.0), gz_h(ell, 0.0);
    // upwind source of face f: (index, kind) with kind -1 interior (index =
    // neighbour cell), -2 isothermal (index = table column), >= 0 specular class
    auto face_src = [&](int64_t f, int32_t *idx, int32_t *kind) {
        const int64_t v = m->face_nbr[f];
        if (v >= 0) {
            *idx = v < nc ? pos_h[v] : (int32_t)v;  // (v >= nc: halo column of a cut face)
            *kind = -1;
        } else {
            const int64_t bf = -1 - v;
            const bool iso = bc->kind[bf] == BTE_BC_ISOTHERMAL;
            *idx = iso ? iso_of[bf] : 0;
            *kind = iso ? -2 : bcls[bf];
        }
    };
    auto code5 = [](int32_t kind) { return kind == -1 ? bte::kCodeInterior : kind == -2 ? bte::kCodeIso : (uint32_t)kind; };
    auto code8 = [](int32_t kind) { return (uint8_t)(kind == -1 ? bte::kCode8Interior : kind == -2 ? bte::kCode8Iso : kind); };
    for (int32_t i = 0; i < nc; ++i) {
        const int64_t c = user_of[i];
        int j = 0;
        for (int64_t f = m->face_offsets[c]; f < m->face_offsets[c + 1]; ++f) {
            if (paired && partner[f] < f) continue;  // "+" face = first of its pair
            const size_t q = (size_t)j * nc + i;
            const double av = m->face_area[f] / m->cell_volume[c];
            gx_h[q] = av * m->face_normal[3 * f + 0];
            gy_h[q] = av * m->face_normal[3 * f + 1];
            gz_h[q] = av * m->face_normal[3 * f + 2];
            int32_t kp = -1, km = -1;
            face_src(f, &nbr_h[q], &kp);
            if (paired) {
                face_src(partner[f], &nbm_h[q], &km);
                const uint32_t bits = code5(kp) | (code5(km) << 5);
                fcode_h[i] = (fcode_h[i] & ~(1023u << (10 * j))) | (bits << (10 * j));
            } else {
                fcode8_h[q] = code8(kp);
            }
            ++j;
        }
        for (; j < mf_t; ++j) {  // padding: zero geometry, self neighbour
            nbr_h[(size_t)j * nc + i] = i;
            if (paired) nbm_h[(size_t)j * nc + i] = i;
        }
    }

    // --- context
    bte_ctx *ctx = new bte_ctx();
    ctx->opt = *o;
    ctx->td = td;
    ctx->rate_now = td && o->rates_now;
    ctx->dim = m->dim;
    ctx->nd = nd;
    ctx->nb = nb;
    ctx->b_lo = b_lo;
    ctx->b_hi = b_hi;
    ctx->nb_loc = nb_loc;
    ctx->mf = mf;
    ctx->mf_t = mf_t;
    ctx->paired = paired;
    if (paired) {  // uniform geometry: g of pair j identical (bitwise) in every cell
        bool uni = true;
        for (int j = 0; j < mf_t && uni; ++j)
            for (int32_t i = 1; i < nc && uni; ++i) {
                const size_t q0 = (size_t)j * nc, q = q0 + i;
                uni = gx_h[q] == gx_h[q0] && gy_h[q] == gy_h[q0] && gz_h[q] == gz_h[q0];
            }
        ctx->uniform_g = uni && !(o->flags & BTE_FLAG_GENERIC_FACES);
        for (int j = 0; j < mf_t; ++j) {
            ctx->gu[j][0] = gx_h[(size_t)j * nc];
            ctx->gu[j][1] = gy_h[(size_t)j * nc];
            ctx->gu[j][2] = gz_h[(size_t)j * nc];
        }
    }
    ctx->nc = nc;
    ctx->ps = ps;
    ctx->n_bcells = n_bcells;
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
    if (o->group) {  // in-process communicator: the ranks are host threads of this process
        std::string e;
        if (!bte::nccl::init_local(&ctx->comm, o->group->g, o->rank, &e)) {
            set_err(&ctx->err, "in-process group: %s", e.c_str());
            return fail(BTE_ENCCL);
        }
        ctx->have_comm = true;
        ctx->graphs_ok = false;  // (its exchanges are host-ordered: launch by launch)
    } else if (o->nccl_unique_id) {  // (world == 1 with an id: a one-rank communicator, same code path)
        std::string e;
        if (!bte::nccl::init(&ctx->comm, o->nccl_unique_id, o->rank, o->world, &e)) {
            set_err(&ctx->err, "NCCL init failed: %s", e.c_str());
            return fail(BTE_ENCCL);
        }
        ctx->have_comm = true;
    }
    ctx->n_parts = n_parts;
    ctx->my_part = my_part;
    ctx->G = G;
    ctx->gband = gband;
    ctx->n_halo = n_halo;
    ctx->gid = lplan.gid;
    if (ctx->have_comm && n_parts == 1) {  // band sharding: the energy goes over the whole communicator
        ctx->bcomm = ctx->comm;
        ctx->have_bcomm = true;
    } else if (ctx->have_comm && G > 1) {  // hybrid: over the ranks of this cell part
        std::string e;
        if (!bte::nccl::split(ctx->comm, my_part, gband, &ctx->bcomm, &e)) {
            set_err(&ctx->err, "NCCL communicator split failed: %s", e.c_str());
            return fail(BTE_ENCCL);
        }
        ctx->have_bcomm = ctx->own_bcomm = true;
    }

    // --- launch plan knobs (band group: measured best on B200)
    ctx->block = block;
    ctx->tma = tma_ok;  // (paired or generic faces)
    if (const char *ev = std::getenv("BTE_NEWTON"))  // warp | thread | lanes4 | lanes8 | lanes16
        ctx->newton_mode = std::strcmp(ev, "warp") == 0 ? 32 : std::strcmp(ev, "thread") == 0 ? 2
                         : std::strncmp(ev, "lanes", 5) == 0 ? std::atoi(ev + 5) : 0;
    if (ctx->newton_mode != 0 && ctx->newton_mode != 2 && ctx->newton_mode != 4 && ctx->newton_mode != 8 &&
        ctx->newton_mode != 16 && ctx->newton_mode != 32)
        ctx->newton_mode = 0;
    // auto band group (measured on B200): the largest group that
    // compiles without spills for the chosen kernel
    const int auto_bg = !paired ? 4 : ctx->uniform_g ? 5 : 3;
    ctx->bg = legal_bg(o->band_group > 0 ? o->band_group : auto_bg, paired);
    if (use_box) {  // one band-row per stage; band_group / dir_chunk size the CTA's work instead
        ctx->box = true;
        ctx->bg = 1;
        for (int a = 0; a < 3; ++a) ctx->bn[a] = bx.n[a], ctx->bgeo[a] = bx.g[a];
        ctx->bz_lo = zs.on ? zs.h_lo : 0;
        ctx->bz_t = bx.n[2] + (zs.on ? zs.h_lo + zs.h_hi : 0);
        ctx->bzside[0] = bx.zside[0];
        ctx->bzside[1] = bx.zside[1];
        ctx->bflat = bx.flat;
        ctx->n_orb = (int)orbs.size();
        // shared memory for 2 CTAs per SM (3-D): ring stages x 12 KB + L x 2 KB energy rows
        // (rate law: 16 KB stages, 5 x 16 + 8 x 2 KB)
        const char *ev = std::getenv("BTE_BOX_STAGES");
        // (2-D, 3 CTAs per SM: 3 stages; orbit chunks of 25 (a C3 slice = 4 chunks).  Measured on B200
        // with the direct stores, round 2: C4 5 stages 7.22 ms, 6 stages 7.63, 4 stages 8.05 -- a
        // deeper ring lets the producer run ahead and the halo rows of the boxes are re-read from
        // DRAM, a shallower one exposes the load latency; C5 5: 52.2 ms, 6: 52.9; C3 3: 0.814 ms,
        // 4: 0.830, 5: 0.840; the rate law's 16 KB stages, C4 with an equilibrium state
        // (tools/sweep_box.py C4+law): 5 stages x 8 layers 7.38 ms, 6 x 4 7.46, 5 x 4 7.77,
        // 6 x 6 8.11, 6 x 8 9.69 (one CTA per SM))
        const int def_stages = bx.flat ? 3 : 5;
        ctx->box_stages = std::max(2, std::min(bte::kBoxMaxStages, ev ? std::atoi(ev) : def_stages));
        if (bx.flat) ctx->box_oc = 25;
        ev = std::getenv("BTE_BOX_L");
        ctx->box_L = std::max(1, std::min<int>(bx.n[2], ev ? std::atoi(ev) : 8));
        ev = std::getenv("BTE_BOX_NBB");
        if (ev) ctx->box_nbb = std::max(1, std::atoi(ev));
        ev = std::getenv("BTE_BOX_OC");
        if (ev) ctx->box_oc = std::max(1, std::atoi(ev));
        CREATE_TRY(box_setup_kernel(ctx));
    }

    // --- slab pool: nb_loc current slabs + n_spare workspace slabs
    ctx->slab_elems = (int64_t)nd * ps;
    const size_t slab_bytes = (size_t)ctx->slab_elems * sizeof(double);
    int n_spare = nb_loc;
    if (o->max_spare_slabs > 0) n_spare = std::min(n_spare, (int)o->max_spare_slabs);
    {
        size_t free_b = 0, total_b = 0;
        CREATE_CUDA(cudaMemGetInfo(&free_b, &total_b));
        const size_t other = (size_t)nc * sizeof(double) * (size_t)(3 * nb_loc + 16) + ell * 48 + (64u << 20);
        const size_t reserve = (size_t)512 << 20;  // (driver / late small allocations; the partial slots are counted)
        // + the energy partial slots, whose count follows the batches of n_spare rows
        auto slot_bytes = [&](int ns) {
            const int keep = ctx->n_spare;
            ctx->n_spare = ns;
            const size_t b = (size_t)count_slots(ctx) * (size_t)nc * sizeof(double);
            ctx->n_spare = keep;
            return b;
        };
        while (n_spare > 1 && (size_t)(nb_loc + n_spare) * slab_bytes + other + slot_bytes(n_spare) + reserve > free_b)
            --n_spare;
        if ((size_t)(nb_loc + n_spare) * slab_bytes + other + slot_bytes(n_spare) > free_b) {
            set_err(&ctx->err, "intensity needs %.1f GB (%d slabs of %.2f GB); %.1f GB free",
                    (nb_loc + n_spare) * slab_bytes / 1e9, nb_loc + n_spare, slab_bytes / 1e9, free_b / 1e9);
            return fail(BTE_ENOMEM);
        }
    }
    // slab rotation: batches of whole band groups (a batch of 11 at group 5 would
    // launch 5 + 5 + 1, and the 1-row tail launch is slow)
    if (n_spare < nb_loc && n_spare >= ctx->bg && o->max_spare_slabs <= 0) n_spare -= n_spare % ctx->bg;
    ctx->n_spare = n_spare;
    while (ctx->bg > n_spare) ctx->bg = std::max(1, legal_bg(ctx->bg - 1, paired));
    ctx->cur_slot.resize(nb_loc);
    ctx->spare_slot.resize(n_spare);
    for (int k = 0; k < nb_loc; ++k) ctx->cur_slot[k] = k;
    for (int k = 0; k < n_spare; ++k) ctx->spare_slot[k] = nb_loc + k;
    CREATE_TRY(dalloc(ctx, &ctx->pool, (size_t)(nb_loc + n_spare) * ctx->slab_elems));
    ctx->pool_cells = ctx->pool + zs.off;

    CREATE_TRY(dalloc(ctx, &ctx->i0, (size_t)nb_loc * nc));
    CREATE_TRY(dalloc(ctx, &ctx->T, (size_t)nc));
    // E padded to world x chunk for the reduce-scatter of the sharded step
    ctx->chunk = (int32_t)((nc64 + G - 1) / G);
    ctx->nc_pad = ctx->chunk * G;
    CREATE_TRY(dalloc(ctx, &ctx->E, (size_t)ctx->nc_pad));
    CREATE_CUDA(cudaMemset(ctx->E, 0, (size_t)ctx->nc_pad * sizeof(double)));
    if (n_halo > 0)  // halo columns are read (times a zero weight) before a direction's first exchange
        CREATE_CUDA(cudaMemsetAsync(ctx->pool, 0, (size_t)(nb_loc + n_spare) * ctx->slab_elems * sizeof(double),
                                    ctx->stream));
    for (const SegPlan &sp : lplan.segs) {  // halo segments: internal columns, direction lists, buffers
        ctx->hsegs.emplace_back();
        HaloSeg &h = ctx->hsegs.back();
        h.part = sp.part;
        h.col0 = nc + sp.col0;
        {  // halo columns relative to pool_cells: after the owned cells, or (z-slab box) the halo layers
            std::vector<int32_t> rc(sp.n_recv_cells);
            const int64_t plane = zs.on ? (int64_t)zs.gbx.n[0] * zs.gbx.n[1] : 0;
            for (int32_t i = 0; i < sp.n_recv_cells; ++i) {
                if (!zs.on) {
                    rc[i] = nc + sp.col0 + i;
                } else {
                    const int64_t gp = zs.grid_of[sp.recv_global[i]];
                    const int64_t layer = gp / plane;
                    rc[i] = (int32_t)((layer - zs.za + zs.h_lo) * plane + gp % plane - zs.off);
                }
            }
            CREATE_TRY(upload(ctx, &h.recv_cols, rc));
        }
        h.n_send_cells = (int32_t)sp.send_local.size();
        h.n_send_dirs = (int32_t)sp.send_dirs.size();
        h.n_recv_cells = sp.n_recv_cells;
        h.n_recv_dirs = (int32_t)sp.recv_dirs.size();
        std::vector<int32_t> cols(sp.send_local.size());
        for (size_t i = 0; i < cols.size(); ++i) cols[i] = pos_h[sp.send_local[i]];
        CREATE_TRY(upload(ctx, &h.send_cells, cols));
        CREATE_TRY(upload(ctx, &h.send_dirs, sp.send_dirs));
        CREATE_TRY(upload(ctx, &h.recv_dirs, sp.recv_dirs));
        CREATE_TRY(dalloc(ctx, &h.sbuf, (size_t)h.n_send() * nb_loc));
        CREATE_TRY(dalloc(ctx, &h.rbuf, (size_t)h.n_recv() * nb_loc));
        ctx->st.halo_bytes += h.n_send() * nb_loc * (int64_t)sizeof(double);
    }
    CREATE_TRY(dalloc(ctx, &ctx->Tg, (size_t)ctx->nc_pad));  // the step's solve writes T^{n+1} here first
    if (ctx->have_bcomm) {
        const char *ev = std::getenv("BTE_SHARD_NEWTON");  // "replicated": all-reduce + replicated solve
        ctx->shard_newton = !(ev && std::strcmp(ev, "replicated") == 0);
        CREATE_TRY(dalloc(ctx, &ctx->Echunk, (size_t)ctx->chunk));
    }
    ctx->staging_elems = std::min<int64_t>((int64_t)nd * nc, std::max<int64_t>(nc, (int64_t)8 << 20));
    CREATE_TRY(dalloc(ctx, &ctx->staging, (size_t)ctx->staging_elems));
    if (ctx->tma && !paired) {  // generic TMA kernel: per-tile staging lists and shared-memory indices
        // per tile: own cells at [0, 256), then the halo cells (interior faces pointing
        // out of the tile) and the boundary-face ghosts at positions of
        // [256, 256 + cap) placed so that each half-warp's upwind loads spread over the
        // 16 bank pairs (fewer shared-memory bank conflicts)
        const int32_t ntiles = (nc + bte::kTile - 1) / bte::kTile;
        std::vector<int32_t> hoff(ntiles + 1, 0), hcell, goff(ntiles + 1, 0), gcol, gcls;
        std::vector<std::vector<size_t>> gface(ntiles);  // face slot q of each ghost
        int32_t smax = 0;
        {
            std::set<int32_t> halo;
            for (int32_t t = 0; t < ntiles; ++t) {
                const int32_t t0 = t * bte::kTile, t1 = std::min(nc, t0 + bte::kTile);
                halo.clear();
                for (int j = 0; j < mf_t; ++j)
                    for (int32_t i = t0; i < t1; ++i) {
                        const size_t q = (size_t)j * nc + i;
                        if (fcode8_h[q] != bte::kCode8Interior) {
                            gface[t].push_back(q);
                            const bool iso = fcode8_h[q] == bte::kCode8Iso;  // Eq. 6: isothermal table column / reflected plane
                            gcol.push_back(iso ? nbr_h[q] : i);
                            gcls.push_back(iso ? -1 : (int32_t)fcode8_h[q]);
                        } else if (nbr_h[q] < t0 || nbr_h[q] >= t0 + bte::kTile) {
                            halo.insert(nbr_h[q]);
                        }
                    }
                // (halo list in ascending cell order: the producer lanes' gathers of
                // neighbouring columns fall into shared 32-byte sectors)
                hcell.insert(hcell.end(), halo.begin(), halo.end());
                hoff[t + 1] = (int32_t)hcell.size();
                goff[t + 1] = (int32_t)gcol.size();
                smax = std::max<int32_t>(smax, (int32_t)halo.size() + (int32_t)gface[t].size());
            }
        }
        if (smax <= bte::kMaxTileStaged) {
            ctx->hstride = bte::kTile + (smax + 31) / 32 * 32;
            if (ctx->hstride <= bte::kTileStagedFixed) ctx->hstride = bte::kTileStagedFixed;  // (compile-time stride)
            const int32_t cap = ctx->hstride - bte::kTile;
            std::vector<uint16_t> sidx_h(ell, 0);
            std::vector<int32_t> hpos(hcell.size()), gpos(gcol.size());
            std::map<int32_t, int32_t> hk;  // halo cell -> its index in the tile's list
            std::vector<std::vector<int32_t>> readers;
            std::vector<int32_t> placed;
            for (int32_t t = 0; t < ntiles; ++t) {
                const int32_t t0 = t * bte::kTile, t1 = std::min(nc, t0 + bte::kTile);
                const int32_t h0 = hoff[t], nh = hoff[t + 1] - h0, g0 = goff[t], ng = goff[t + 1] - g0;
                hk.clear();
                for (int32_t k = 0; k < nh; ++k) hk[hcell[h0 + k]] = k;
                int deg[bte::kTile / 16][16] = {};  // upwind reads per (half-warp, bank class)
                readers.assign(nh + ng, {});
                for (int j = 0; j < mf_t; ++j)
                    for (int32_t i = t0; i < t1; ++i) {
                        const size_t q = (size_t)j * nc + i;
                        const int32_t H = (i - t0) >> 4, v = nbr_h[q];
                        if (fcode8_h[q] != bte::kCode8Interior) continue;
                        if (v >= t0 && v < t0 + bte::kTile) {
                            sidx_h[q] = (uint16_t)(v - t0);
                            ++deg[H][(v - t0) & 15];
                        } else {
                            auto &r = readers[hk[v]];
                            if (std::find(r.begin(), r.end(), H) == r.end()) r.push_back(H);
                        }
                    }
                for (int32_t g = 0; g < ng; ++g) readers[nh + g].push_back((int32_t)((gface[t][g] % nc) - t0) >> 4);
                place_staged(readers, deg, bte::kTile, cap, placed);
                for (int32_t k = 0; k < nh + ng; ++k) {
                    if (k < nh) hpos[h0 + k] = placed[k]; else gpos[g0 + k - nh] = placed[k];
                }
                for (int j = 0; j < mf_t; ++j)
                    for (int32_t i = t0; i < t1; ++i) {
                        const size_t q = (size_t)j * nc + i;
                        const int32_t v = nbr_h[q];
                        if (fcode8_h[q] == bte::kCode8Interior && (v < t0 || v >= t0 + bte::kTile))
                            sidx_h[q] = (uint16_t)hpos[h0 + hk[v]];
                    }
                for (int32_t g = 0; g < ng; ++g) sidx_h[gface[t][g]] = (uint16_t)gpos[g0 + g];
            }
            // faces of each cell permuted among its slots against the remaining conflicts
            std::vector<uint8_t> perm;
            const auto wf = order_face_slots(sidx_h, nc, mf_t, perm);
            if (std::getenv("BTE_DEBUG_SLOTS"))
                std::fprintf(stderr, "bte: upwind shared-load wavefronts (all half-warps, slots) %lld -> %lld\n",
                             (long long)wf.first, (long long)wf.second);
            {
                std::vector<int32_t> t_nbr(mf_t);
                std::vector<uint8_t> t_code(mf_t);
                std::vector<double> t_g(3 * mf_t);
                for (int32_t i = 0; i < nc; ++i) {
                    for (int j = 0; j < mf_t; ++j) {
                        const size_t q = (size_t)perm[(size_t)i * mf_t + j] * nc + i;
                        t_nbr[j] = nbr_h[q];
                        t_code[j] = fcode8_h[q];
                        t_g[3 * j] = gx_h[q];
                        t_g[3 * j + 1] = gy_h[q];
                        t_g[3 * j + 2] = gz_h[q];
                    }
                    for (int j = 0; j < mf_t; ++j) {
                        const size_t q = (size_t)j * nc + i;
                        nbr_h[q] = t_nbr[j];
                        fcode8_h[q] = t_code[j];
                        gx_h[q] = t_g[3 * j];
                        gy_h[q] = t_g[3 * j + 1];
                        gz_h[q] = t_g[3 * j + 2];
                    }
                }
            }
            // the kernel indexes shared memory with these lists: check them (after the face-slot order: every
            // staged index inside the row, each tile's halo / ghost positions distinct and
            // inside [kTile, hstride), a face's index = its upwind value's position)
            {
                std::vector<int32_t> owner(cap);
                for (int32_t t = 0; t < ntiles; ++t) {
                    const int32_t t0 = t * bte::kTile, t1 = std::min(nc, t0 + bte::kTile);
                    std::fill(owner.begin(), owner.end(), -1);
                    bool ok = true;
                    for (int32_t k = hoff[t]; k < hoff[t + 1] && ok; ++k) {
                        const int32_t p = hpos[k] - bte::kTile;
                        ok = p >= 0 && p < cap && owner[p] < 0;
                        if (ok) owner[p] = k;
                    }
                    for (int32_t g = goff[t]; g < goff[t + 1] && ok; ++g) {
                        const int32_t p = gpos[g] - bte::kTile;
                        ok = p >= 0 && p < cap && owner[p] < 0;
                        if (ok) owner[p] = (int32_t)hcell.size() + g;
                    }
                    for (int j = 0; j < mf_t && ok; ++j)
                        for (int32_t i = t0; i < t1 && ok; ++i) {
                            const size_t q = (size_t)j * nc + i;
                            const int32_t v = nbr_h[q], s = sidx_h[q];
                            if (fcode8_h[q] != bte::kCode8Interior)
                                ok = s >= bte::kTile && s < ctx->hstride && owner[s - bte::kTile] >= (int32_t)hcell.size();
                            else if (v >= t0 && v < t0 + bte::kTile)  // (incl. halo columns >= nc of a cell part)
                                ok = s == v - t0 && v < ctx->ps;
                            else
                                ok = s >= bte::kTile && s < ctx->hstride && owner[s - bte::kTile] >= 0 &&
                                     owner[s - bte::kTile] < (int32_t)hcell.size() && hcell[owner[s - bte::kTile]] == v;
                        }
                    if (!ok) {
                        set_err(&ctx->err, "internal: inconsistent shared-memory staging lists of tile %d", t);
                        return fail(BTE_EINVAL);
                    }
                }
            }
            CREATE_TRY(upload(ctx, &ctx->hl_off, hoff));
            CREATE_TRY(upload(ctx, &ctx->hl_cell, hcell));
            CREATE_TRY(upload(ctx, &ctx->hl_pos, hpos));
            CREATE_TRY(upload(ctx, &ctx->bl_off, goff));
            CREATE_TRY(upload(ctx, &ctx->bl_col, gcol));
            CREATE_TRY(upload(ctx, &ctx->bl_cls, gcls));
            CREATE_TRY(upload(ctx, &ctx->bl_pos, gpos));
            CREATE_TRY(upload(ctx, &ctx->sidx, sidx_h));
        } else {
            ctx->tma = false;  // too much to stage per tile: the register kernel
        }
    }
    // energy partial slots (after the kernel choice: the launch segments depend on it)
    CREATE_TRY(dalloc(ctx, &ctx->part, (size_t)count_slots(ctx) * nc));
    CREATE_TRY(upload(ctx, &ctx->d_cur_slot, ctx->cur_slot));
    CREATE_TRY(upload(ctx, &ctx->nbr, nbr_h));
    CREATE_TRY(upload(ctx, &ctx->nbm, nbm_h));
    CREATE_TRY(upload(ctx, &ctx->fcode, fcode_h));
    CREATE_TRY(upload(ctx, &ctx->fcode8, fcode8_h));
    CREATE_TRY(upload(ctx, &ctx->gx, gx_h));
    CREATE_TRY(upload(ctx, &ctx->gy, gy_h));
    CREATE_TRY(upload(ctx, &ctx->gz, gz_h));
    CREATE_TRY(upload(ctx, &ctx->pos, pos_h));
    ctx->identity_order = true;
    for (int32_t i = 0; i < nc && ctx->identity_order; ++i) ctx->identity_order = pos_h[i] == i;
    CREATE_TRY(upload(ctx, &ctx->refl, refl_h));
    CREATE_TRY(upload(ctx, &ctx->twall, twall_h));
    std::vector<double4> dirs_h(nd);
    for (int d = 0; d < nd; ++d) dirs_h[d] = make_double4(dr->s[3 * d], dr->s[3 * d + 1], dr->s[3 * d + 2], dr->w[d]);
    CREATE_TRY(upload(ctx, &ctx->dirs, dirs_h));
    ctx->h_inv_tau.assign(inv_tau.begin() + b_lo, inv_tau.begin() + b_hi);
    ctx->h_vg.assign(bd->vg + b_lo, bd->vg + b_hi);
    ctx->h_cw.assign(cw.begin() + b_lo, cw.begin() + b_hi);
    CREATE_TRY(upload(ctx, &ctx->cw_loc, ctx->h_cw));
    CREATE_TRY(upload(ctx, &ctx->Cb, Cb_all));
    CREATE_TRY(upload(ctx, &ctx->theta, theta));
    {  // temperature-equation terms (constant weights only: not R2 with the rate law)
        std::vector<double> th_t, k_t, ic_t;
        std::vector<int32_t> rep_t;
        if (!(td && o->temp_rule == 0)) {
            std::vector<int> term_of(nb, -1);
            for (int b = 0; b < nb; ++b) {
                for (size_t j = 0; j < th_t.size() && term_of[b] < 0; ++j)
                    if (th_t[j] == theta[b]) term_of[b] = (int)j;
                if (term_of[b] < 0) {
                    term_of[b] = (int)th_t.size();
                    th_t.push_back(theta[b]);
                    rep_t.push_back(b);
                    ic_t.push_back(1.0 / Cb_all[b]);
                    k_t.push_back(0.0);
                }
            }
            for (int b = 0; b < nb; ++b) k_t[term_of[b]] += cw[b] * Cb_all[b];
        }
        ctx->n_terms = (int)th_t.size();
        if (ctx->n_terms > 0) {  // rows of a term as a list: rep[j], nrow[rep[j]], ...
            std::vector<int32_t> nrow(nb, -1), last(ctx->n_terms, -1);
            for (int b = 0; b < nb; ++b) {
                int j = 0;
                while (th_t[j] != theta[b]) ++j;
                if (last[j] >= 0) nrow[last[j]] = b;
                last[j] = b;
            }
            CREATE_TRY(upload(ctx, &ctx->t_nrow, nrow));
        }
        CREATE_TRY(upload(ctx, &ctx->t_th, th_t));
        CREATE_TRY(upload(ctx, &ctx->t_k, k_t));
        CREATE_TRY(upload(ctx, &ctx->t_ic, ic_t));
        CREATE_TRY(upload(ctx, &ctx->t_rep, rep_t));
    }
    CREATE_TRY(upload(ctx, &ctx->cw_all, cw));
    CREATE_TRY(dalloc(ctx, &ctx->i0w, (size_t)nb_loc * std::max(1, ctx->n_iso)));
    CREATE_TRY(dalloc(ctx, &ctx->d_iter_max, 1));
    CREATE_TRY(dalloc(ctx, &ctx->fresh, (size_t)nc));
    CREATE_TRY(dalloc(ctx, &ctx->d_flags, 4));
    ctx->d_fail = ctx->d_flags;
    ctx->d_halt = ctx->d_flags + 1;
    ctx->d_done = ctx->d_flags + 2;
    CREATE_TRY(dalloc(ctx, &ctx->d_smax, 1));
    CREATE_CUDA(cudaMemsetAsync(ctx->d_iter_max, 0, sizeof(int32_t), ctx->stream));
    CREATE_CUDA(cudaMemsetAsync(ctx->d_flags, 0, 4 * sizeof(int32_t), ctx->stream));
    CREATE_CUDA(cudaMemsetAsync(ctx->d_smax, 0, sizeof(unsigned long long), ctx->stream));

    // --- initial state: T = t_init, I = I0_b(t_init); isothermal table; dt bound
    {
        std::vector<double> T0(nc, o->t_init);
        CREATE_CUDA(cudaMemcpy(ctx->T, T0.data(), nc * sizeof(double), cudaMemcpyHostToDevice));
        const int tb = 256;
        const int gb = (nc + tb - 1) / tb;
        bte::i0_table_kernel<<<gb, tb, 0, ctx->stream>>>(ctx->T, nc, b_lo, nb_loc, ctx->Cb, ctx->theta, ctx->i0);
        bte::equilibrium_kernel<<<dim3(std::min<int64_t>(4096, ((int64_t)nd * nc + tb - 1) / tb), nb_loc), tb, 0,
                                  ctx->stream>>>(ctx->pool_cells, ctx->d_cur_slot, ctx->slab_elems, ps, nd, nc, ctx->i0);
        if (ctx->n_iso > 0)
            bte::i0w_kernel<<<(ctx->n_iso + tb - 1) / tb, tb, 0, ctx->stream>>>(ctx->twall, ctx->n_iso, b_lo, nb_loc,
                                                                               ctx->Cb, ctx->theta, ctx->i0w);
        if (m->dim == 2)
            bte::outflow_max_kernel<2><<<gb, tb, 0, ctx->stream>>>(nc, mf_t, paired, nd, ctx->gx, ctx->gy, ctx->gz,
                                                                  ctx->dirs, ctx->d_smax);
        else
            bte::outflow_max_kernel<3><<<gb, tb, 0, ctx->stream>>>(nc, mf_t, paired, nd, ctx->gx, ctx->gy, ctx->gz,
                                                                  ctx->dirs, ctx->d_smax);
        CREATE_CUDA(cudaGetLastError());
        if (ctx->have_comm && n_parts > 1) {  // the bound of the whole mesh on every rank (S_max >= 0: bits = value)
            std::string e;
            if (!bte::nccl::allreduce_max_f64(ctx->comm, reinterpret_cast<double *>(ctx->d_smax), 1, ctx->stream, &e)) {
                set_err(&ctx->err, "NCCL all-reduce (max) failed: %s", e.c_str());
                return fail(BTE_ENCCL);
            }
        }
        unsigned long long bits = 0;
        CREATE_CUDA(cudaMemcpyAsync(&bits, ctx->d_smax, sizeof bits, cudaMemcpyDeviceToHost, ctx->stream));
        CREATE_CUDA(cudaStreamSynchronize(ctx->stream));
        std::memcpy(&ctx->s_max, &bits, sizeof(double));
        ctx->h_inv_tau_all = inv_tau;
        ctx->h_vg_all.assign(bd->vg, bd->vg + nb);
        ctx->t_hi = o->t_init;
        for (int64_t f = 0; f < bc->n_bfaces; ++f)
            if (bc->kind[f] == BTE_BC_ISOTHERMAL) ctx->t_hi = std::max(ctx->t_hi, bc->t_wall[f]);
        if (td) {  // rate law tables: Tr = T = t_init, both halves at t_init
            ctx->h_ra.assign(bd->rate_a, bd->rate_a + nb);
            ctx->h_rb.assign(bd->rate_b, bd->rate_b + nb);
            ctx->h_rth.assign(bd->rate_theta, bd->rate_theta + nb);
            std::vector<double> iv(nb);
            for (int b = 0; b < nb; ++b) iv[b] = 1.0 / bd->vg[b];
            CREATE_TRY(upload(ctx, &ctx->d_ra, ctx->h_ra));
            CREATE_TRY(upload(ctx, &ctx->d_rb, ctx->h_rb));
            CREATE_TRY(upload(ctx, &ctx->d_rth, ctx->h_rth));
            CREATE_TRY(upload(ctx, &ctx->d_inv_v, iv));
            CREATE_TRY(dalloc(ctx, &ctx->rates, (size_t)2 * nb_loc * nc));
            CREATE_TRY(dalloc(ctx, &ctx->Tr, (size_t)nc));
            CREATE_TRY(refresh_i0(ctx));
        }
        update_dt_bound(ctx);
    }
    if (ctx->box) {  // orbit table, grid-axis directions, isothermal side tables, tensor maps
        CREATE_TRY(upload(ctx, &ctx->orb, orbs));
        std::vector<double4> db(nd);
        for (int d = 0; d < nd; ++d) {
            const double *sd = dr->s + 3 * d;
            db[d] = make_double4(sd[bx.ax[0]], sd[bx.ax[1]], sd[bx.ax[2]], dr->w[d]);
        }
        CREATE_TRY(upload(ctx, &ctx->dirs_box, db));
        const int64_t nside = bx.flat ? (int64_t)bx.n[0] : (int64_t)bx.n[0] * bx.n[1];
        std::vector<int32_t> col(2 * nside, -1);
        for (int sd = 0; sd < 2; ++sd)
            if (bx.zside[sd] == 0)
                for (int64_t i = 0; i < nside; ++i) col[sd * nside + i] = iso_of[bx.zbface[sd][i]];
        CREATE_TRY(upload(ctx, &ctx->side_col, col));
        CREATE_TRY(dalloc(ctx, &ctx->side_tab, (size_t)nb_loc * 2 * nside));
        bte::side_table_kernel<<<256, 256, 0, ctx->stream>>>(ctx->i0w, ctx->n_iso, ctx->side_col, (int)(2 * nside),
                                                            nb_loc, ctx->side_tab);
        CREATE_CUDA(cudaGetLastError());
        const uint64_t n0 = bx.n[0], n1 = bx.n[1], n2 = bx.n[2];
        const uint64_t dpool[5] = {n0, n1, (uint64_t)ctx->bz_t, (uint64_t)nd, (uint64_t)(nb_loc + n_spare)};
        const uint64_t spool[4] = {n0 * 8, n0 * n1 * 8, (uint64_t)ps * 8, (uint64_t)ctx->slab_elems * 8};
        const uint32_t bin[5] = {bte::kBoxBX, bte::kBoxBY, 1, 1, 1}, bout[5] = {bte::kBoxTX, bte::kBoxTY, 1, 1, 1};
        const uint64_t di0[4] = {n0, n1, n2, (uint64_t)nb_loc}, si0[3] = {n0 * 8, n0 * n1 * 8, (uint64_t)nc * 8};
        const uint64_t dsd[4] = {n0, n1, 2, (uint64_t)nb_loc}, ssd[3] = {n0 * 8, n0 * n1 * 8, 2 * n0 * n1 * 8};
        // 2-D: the wall rows of grid axis 1 as {n0, 2, nb_loc}, one 32-cell row per load
        const uint64_t dsf[3] = {n0, 2, (uint64_t)nb_loc}, ssf[2] = {n0 * 8, 2 * n0 * 8};
        const uint32_t bsf[3] = {bte::kBoxTX, 1, 1};
        const uint64_t drt[5] = {n0, n1, n2, (uint64_t)nb_loc, 2},
                       srt[4] = {n0 * 8, n0 * n1 * 8, (uint64_t)nc * 8, (uint64_t)nb_loc * nc * 8};
        if (!encode_map(&ctx->tm_in, ctx->pool, 5, dpool, spool, bin) ||
            !encode_map(&ctx->tm_out, ctx->pool, 5, dpool, spool, bout) ||
            !encode_map(&ctx->tm_i0, ctx->i0, 4, di0, si0, bout) ||
            !(bx.flat ? encode_map(&ctx->tm_side, ctx->side_tab, 3, dsf, ssf, bsf)
                      : encode_map(&ctx->tm_side, ctx->side_tab, 4, dsd, ssd, bin)) ||
            !encode_map(&ctx->tm_rate, ctx->td ? ctx->rates : ctx->i0, ctx->td ? 5 : 4, ctx->td ? drt : di0,
                        ctx->td ? srt : si0, bout)) {
            set_err(&ctx->err, "cuTensorMapEncodeTiled failed for the box kernel maps");
            return fail(BTE_ECUDA);
        }
        CREATE_CUDA(cudaStreamSynchronize(ctx->stream));
    }
    {
        const int64_t hb = ctx->st.halo_bytes;
        std::memset(&ctx->st, 0, sizeof ctx->st);
        ctx->st.halo_bytes = hb;
    }
    ctx->st.spare_slabs = n_spare;
    ctx->st.n_interior_cells = nc - n_bcells;
    ctx->st.band_group = ctx->box ? plan_box(ctx, std::min(ctx->n_spare, nb_loc)).nbb : ctx->bg;
    ctx->st.block_threads = ctx->box ? bte::kBoxThreads : ctx->block;
    *out = ctx;
    return BTE_OK;
#undef CREATE_TRY
#undef CREATE_CUDA
}

}  // extern "C"
