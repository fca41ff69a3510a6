/*
 * bte_oracle.c -- CPU ORACLE (test infrastructure only; see bte_oracle.h).
 *
 * Plain loops in the paper's order and notation.  Nothing here is blocked,
 * fused or reordered beyond what the equations state.  The only concession to
 * run time is an OpenMP pragma over the independent cell loops (per-cell
 * arithmetic is unchanged, so results do not depend on the thread count).
 */
#include "bte_oracle.h"

#include <math.h>
#include <stdlib.h>
#include <string.h>

/* CODATA 2018 exact/defining values (external). */
#define ORACLE_HBAR 1.054571817e-34 /* J s */
#define ORACLE_KB 1.380649e-23      /* J / K */

/* ------------------------------------------------------------------ physics */

/* I0_b(T) = C_b / (exp(theta_b/T) - 1), theta_b = hbar omega_b / kB.
 * Bose-Einstein equilibrium per direction (L498-499; form per SURVEY 8(c) #4).
 * expm1 because low bands have theta/T ~ 0.02. */
double oracle_I0(double C, double omega, double T) {
    double theta = ORACLE_HBAR * omega / ORACLE_KB;
    return C / expm1(theta / T);
}

/* dI0/dT = C (theta/T^2) e^x / (e^x - 1)^2, x = theta/T, written as
 * I0 (x/T) (1 + 1/expm1(x)) so that it stays finite for large x. */
static double oracle_dI0dT(double C, double omega, double T) {
    double theta = ORACLE_HBAR * omega / ORACLE_KB;
    double x = theta / T;
    double em1 = expm1(x);
    return (C / em1) * (x / T) * (1.0 + 1.0 / em1);
}

/* Scattering rate 1/tau_b (Eq. 5's 1/tau_b, L549).  Constant: 1/tau_b (tau =
 * +inf gives 0).  Temperature-dependent (N1, L666-669): the law
 *   1/tau_b(T) = a_b + b_b T exp(-theta_b / T)
 * (impurity-like + Umklapp-like terms; the form is external)
 * at the rate temperature Tr. */
double oracle_rate(const oracle_problem *p, int32_t b, double Tr) {
    if (p->rate_a) return p->rate_a[b] + p->rate_b[b] * Tr * exp(-p->rate_theta[b] / Tr);
    if (isinf(p->tau[b])) return 0.0;
    return 1.0 / p->tau[b];
}

/* Temperature weight c_b:
 * R2 (default): c_b = (1/tau_b) / v_b  -- tau = +inf gives 0;
 * R1:           c_b = 1/v_b. */
double oracle_weight_at(const oracle_problem *p, int32_t b, double Tr) {
    if (p->temp_rule == 1 || p->temp_rule == 2) return 1.0 / p->vg[b];
    if (!p->rate_a) {
        if (isinf(p->tau[b])) return 0.0;
        return 1.0 / (p->vg[b] * p->tau[b]);
    }
    return oracle_rate(p, b, Tr) / p->vg[b];
}

double oracle_weight(const oracle_problem *p, int32_t b) { return oracle_weight_at(p, b, NAN); }

/* ------------------------------------------------------------------ Eq. 6 map */

int oracle_reflection_map(const oracle_problem *p, int32_t *r) {
    const int32_t nd = p->n_dirs;
    for (int64_t f = 0; f < p->n_bfaces * nd; ++f) r[f] = -1;
    /* boundary face id -> its normal: walk the CSR face lists */
    for (int64_t c = 0; c < p->n_cells; ++c) {
        for (int64_t f = p->face_offsets[c]; f < p->face_offsets[c + 1]; ++f) {
            if (p->face_nbr[f] >= 0) continue;
            int64_t bf = -1 - p->face_nbr[f];
            if (p->bkind[bf] != 1) continue;
            const double *n = &p->face_normal[3 * f];
            for (int32_t d = 0; d < nd; ++d) {
                const double *s = &p->s[3 * d];
                double mu = s[0] * n[0] + s[1] * n[1] + s[2] * n[2];
                double rs[3] = {s[0] - 2.0 * mu * n[0], s[1] - 2.0 * mu * n[1],
                                s[2] - 2.0 * mu * n[2]};
                int32_t found = -1;
                for (int32_t e = 0; e < nd; ++e) {
                    const double *t = &p->s[3 * e];
                    if (fabs(t[0] - rs[0]) <= 1e-10 && fabs(t[1] - rs[1]) <= 1e-10 &&
                        fabs(t[2] - rs[2]) <= 1e-10) {
                        found = e;
                        break;
                    }
                }
                if (found < 0) return ORACLE_EINVAL;
                r[bf * nd + d] = found;
            }
        }
    }
    return ORACLE_OK;
}

/* ------------------------------------------------------------------ Eq. 3 / 5 */

/* I^n accessor: the full update is written once against it. */
typedef double (*oracle_in_fn)(const void *ctx, int32_t b, int32_t d, int64_t c);

typedef struct {
    const double *I;
    int32_t nd;
    int64_t nc;
} field_ctx;

static double field_in(const void *vctx, int32_t b, int32_t d, int64_t c) {
    const field_ctx *x = (const field_ctx *)vctx;
    return x->I[((int64_t)b * x->nd + d) * x->nc + c];
}

/* One unknown I_{d,b} of cell c advanced by one forward-Euler step.
 *   u = u0 + dt (s(u0) - (1/V) sum_i A_i f_i(u0))          Eq. 3 (L292)
 *   s(u0) = (I0_b(T_c) - I_{d,b}) / tau_b                   Eq. 5 (L546-553)
 *   f_i = |v_g|_b (s_d . n_i) I_hat_i                        Eq. 5 surface term
 *   I_hat_i = I (c)            if s_d.n_i > 0                upwind (L264-267)
 *           = I (nbr)          interior face, s_d.n_i <= 0
 *           = I0_b(T_wall)     isothermal boundary face      Eq. 6
 *           = I_{r,b} (c)      symmetric boundary face       Eq. 6 (old level)
 */
static double update_one(const oracle_problem *p, const int32_t *r, const double *T, const double *Tr,
                         oracle_in_fn In, const void *ctx, double dt, int32_t b, int32_t d,
                         int64_t c) {
    const double *s = &p->s[3 * d];
    const double Ic = In(ctx, b, d, c);
    double F = 0.0;
    for (int64_t f = p->face_offsets[c]; f < p->face_offsets[c + 1]; ++f) {
        const double *n = &p->face_normal[3 * f];
        double mu = s[0] * n[0] + s[1] * n[1] + s[2] * n[2];
        double Ihat;
        if (mu > 0.0) {
            Ihat = Ic;
        } else if (p->face_nbr[f] >= 0) {
            Ihat = In(ctx, b, d, p->face_nbr[f]);
        } else {
            int64_t bf = -1 - p->face_nbr[f];
            if (p->bkind[bf] == 0)
                Ihat = oracle_I0(p->C[b], p->omega[b], p->t_wall[bf]);
            else
                Ihat = In(ctx, b, r[bf * p->n_dirs + d], c);
        }
        F += p->face_area[f] * mu * Ihat;
    }
    double inv_tau = oracle_rate(p, b, Tr ? Tr[c] : NAN);
    double I0 = oracle_I0(p->C[b], p->omega[b], T[c]);
    return Ic + dt * ((I0 - Ic) * inv_tau - p->vg[b] * F / p->cell_volume[c]);
}

void oracle_update_intensity(const oracle_problem *p, const int32_t *r, const double *T, const double *Tr,
                             const double *I, double *Inew, double dt, int32_t b_lo, int32_t b_hi) {
    field_ctx ctx = {I, p->n_dirs, p->n_cells};
    const int64_t nc = p->n_cells;
    for (int32_t b = b_lo; b < b_hi; ++b)
        for (int32_t d = 0; d < p->n_dirs; ++d) {
            double *out = &Inew[((int64_t)b * p->n_dirs + d) * nc];
#pragma omp parallel for schedule(static)
            for (int64_t c = 0; c < nc; ++c)
                out[c] = update_one(p, r, T, Tr, field_in, &ctx, dt, b, d, c);
        }
}

/* ------------------------------------------------------------------ energy */

/* E_c = sum_b c_b sum_d w_d I_{d,b}(c): "integrating the phonon intensity over
 * all directions and bands" (L415-418), weights per SURVEY 8(c) #5. */
void oracle_energy(const oracle_problem *p, const double *I, const double *Tr, int32_t b_lo, int32_t b_hi,
                   double *E) {
    const int64_t nc = p->n_cells;
    const int32_t nd = p->n_dirs;
#pragma omp parallel for schedule(static)
    for (int64_t c = 0; c < nc; ++c) {
        double e = 0.0;
        for (int32_t b = b_lo; b < b_hi; ++b) {
            double sb = 0.0;
            for (int32_t d = 0; d < nd; ++d) sb += p->w[d] * I[((int64_t)b * nd + d) * nc + c];
            e += oracle_weight_at(p, b, Tr ? Tr[c] : NAN) * sb;
        }
        E[c] = e;
    }
}

/* ------------------------------------------------------------------ temperature */

/* g(T) = W sum_b c_b I0_b(T) - E, strictly increasing in T;
 * the weights are taken at the cell's rate temperature Tr (fixed in the solve). */
static double g_of(const oracle_problem *p, double W, double E, double Tr, double T) {
    double g = 0.0;
    for (int32_t b = 0; b < p->n_bands; ++b) g += oracle_weight_at(p, b, Tr) * oracle_I0(p->C[b], p->omega[b], T);
    return W * g - E;
}

static double gprime_of(const oracle_problem *p, double W, double Tr, double T) {
    double g = 0.0;
    for (int32_t b = 0; b < p->n_bands; ++b)
        g += oracle_weight_at(p, b, Tr) * oracle_dI0dT(p->C[b], p->omega[b], T);
    return W * g;
}

/* Bisection on a bracket grown from T0 by halving/doubling. */
static int bisect(const oracle_problem *p, double W, double E, double Tr, double T0, double *T) {
    double lo = T0, hi = T0;
    int k = 0;
    while (g_of(p, W, E, Tr, lo) > 0.0 && k++ < 2000) lo *= 0.5;
    k = 0;
    while (g_of(p, W, E, Tr, hi) < 0.0 && k++ < 2000) hi *= 2.0;
    if (!(g_of(p, W, E, Tr, lo) <= 0.0 && g_of(p, W, E, Tr, hi) >= 0.0)) return ORACLE_ENOCONV;
    for (k = 0; k < 400 && (hi - lo) > p->newton_rtol * hi; ++k) {
        double mid = 0.5 * (lo + hi);
        if (g_of(p, W, E, Tr, mid) < 0.0) lo = mid; else hi = mid;
    }
    *T = 0.5 * (lo + hi);
    return ORACLE_OK;
}

/* Newton from the previous temperature:
 *   T <- T - g(T)/g'(T) until |dT| <= rtol T, at most maxit iterations;
 *   a non-positive or non-finite iterate, or no convergence, falls back to
 *   bisection. */
static int solve_cell(const oracle_problem *p, double W, double E, double Tr, double *T, int32_t *iters) {
    double Tc = *T;
    if (!(E > 0.0) || !isfinite(E)) return ORACLE_ENOCONV;
    if (p->temp_rule == 2) {
        /* R3: T' = T + (E - E_eq(T)) / C(T), C = dE_eq/dT -- one linearised
         * "first law" step from the previous temperature (L413-415). */
        double Tn = Tc - g_of(p, W, E, Tr, Tc) / gprime_of(p, W, Tr, Tc);
        if (!(Tn > 0.0) || !isfinite(Tn)) return ORACLE_ENOCONV;
        *T = Tn;
        if (iters) *iters = 1;
        return ORACLE_OK;
    }
    for (int32_t it = 1; it <= p->newton_maxit; ++it) {
        double delta = g_of(p, W, E, Tr, Tc) / gprime_of(p, W, Tr, Tc);
        double Tn = Tc - delta;
        if (!(Tn > 0.0) || !isfinite(Tn)) break;
        Tc = Tn;
        if (fabs(delta) <= p->newton_rtol * Tc) {
            *T = Tc;
            if (iters) *iters = it;
            return ORACLE_OK;
        }
    }
    if (iters) *iters = -1;
    return bisect(p, W, E, Tr, *T, T);
}

int oracle_newton(const oracle_problem *p, const double *E, const double *Tr, double *T, int32_t *iters) {
    double W = 0.0;
    for (int32_t d = 0; d < p->n_dirs; ++d) W += p->w[d];
    int status = ORACLE_OK;
#pragma omp parallel for schedule(static)
    for (int64_t c = 0; c < p->n_cells; ++c) {
        int32_t it = 0;
        int rc = solve_cell(p, W, E[c], Tr ? Tr[c] : NAN, &T[c], &it);
        if (iters) iters[c] = it;
        if (rc != ORACLE_OK) {
#pragma omp critical
            status = rc;
        }
    }
    return status;
}

void oracle_equilibrium(const oracle_problem *p, const double *T, int32_t b_lo, int32_t b_hi, double *I) {
    const int64_t nc = p->n_cells;
    for (int32_t b = b_lo; b < b_hi; ++b)
        for (int32_t d = 0; d < p->n_dirs; ++d) {
            double *out = &I[((int64_t)(b - b_lo) * p->n_dirs + d) * nc];
#pragma omp parallel for schedule(static)
            for (int64_t c = 0; c < nc; ++c) out[c] = oracle_I0(p->C[b], p->omega[b], T[c]);
        }
}

/* ------------------------------------------------------------------ steps */

int oracle_run(const oracle_problem *p, double dt, int64_t nsteps, double *I, double *T, double *Tr) {
    const int64_t n = (int64_t)p->n_bands * p->n_dirs * p->n_cells;
    int32_t *r = (int32_t *)malloc(sizeof(int32_t) * (size_t)(p->n_bfaces * p->n_dirs + 1));
    double *Inew = (double *)malloc(sizeof(double) * (size_t)(n + 1));
    double *E = (double *)malloc(sizeof(double) * (size_t)(p->n_cells + 1));
    int rc = (r && Inew && E) ? oracle_reflection_map(p, r) : ORACLE_EINVAL;
    if (p->rate_a && !Tr) rc = ORACLE_EINVAL;
    for (int64_t step = 0; step < nsteps && rc == ORACLE_OK; ++step) {
        /* Finch loop (L357-372): u_new from u; then the post-step temperature
         * update (L707-716), where I0 and tau become those of the new state
         * (L666-669; tau one step behind, reading 22, unless rates_now: tau
         * of the step's own temperature, reading 26); then u = u_new. */
        if (Tr && p->rates_now) memcpy(Tr, T, sizeof(double) * (size_t)p->n_cells);
        oracle_update_intensity(p, r, T, Tr, I, Inew, dt, 0, p->n_bands);
        if (Tr) memcpy(Tr, T, sizeof(double) * (size_t)p->n_cells);
        oracle_energy(p, Inew, Tr, 0, p->n_bands, E);
        rc = oracle_newton(p, E, Tr, T, NULL);
        memcpy(I, Inew, sizeof(double) * (size_t)n);
    }
    free(r);
    free(Inew);
    free(E);
    return rc;
}

/* ------------------------------------------------------------------ sampled */

typedef struct {
    const oracle_problem *p;
    const double *T0;
} eq_ctx;

static double eq_in(const void *vctx, int32_t b, int32_t d, int64_t c) {
    const eq_ctx *x = (const eq_ctx *)vctx;
    (void)d;
    return oracle_I0(x->p->C[b], x->p->omega[b], x->T0[c]);
}

int oracle_step_cells_equilibrium(const oracle_problem *p, const int32_t *r, const double *T0,
                                  const int64_t *cells, int64_t n_sel, double dt,
                                  double *Inew_sel, double *T1_sel) {
    eq_ctx ctx = {p, T0};
    const int32_t nb = p->n_bands, nd = p->n_dirs;
    double W = 0.0;
    for (int32_t d = 0; d < nd; ++d) W += p->w[d];
    int status = ORACLE_OK;
#pragma omp parallel for schedule(dynamic)
    for (int64_t k = 0; k < n_sel; ++k) {
        const int64_t c = cells[k];
        double *out = &Inew_sel[k * nb * nd];
        for (int32_t b = 0; b < nb; ++b)
            for (int32_t d = 0; d < nd; ++d)
                out[b * nd + d] = update_one(p, r, T0, T0, eq_in, &ctx, dt, b, d, c);
        double e = 0.0;
        for (int32_t b = 0; b < nb; ++b) {
            double sb = 0.0;
            for (int32_t d = 0; d < nd; ++d) sb += p->w[d] * out[b * nd + d];
            e += oracle_weight_at(p, b, T0[c]) * sb;
        }
        double Tc = T0[c];
        int rc = solve_cell(p, W, e, T0[c], &Tc, NULL);
        T1_sel[k] = Tc;
        if (rc != ORACLE_OK) {
#pragma omp critical
            status = rc;
        }
    }
    return status;
}

/* ------------------------------------------------------------------ subsets */

typedef struct {
    const double *I; /* [nb][nd][n_sub] */
    const int64_t *sub;
    int64_t n_sub;
    int32_t nd;
    int missing;     /* set when a requested cell is not in sub */
} subset_ctx;

static int64_t subset_index(const int64_t *sub, int64_t n, int64_t c) {
    int64_t lo = 0, hi = n;
    while (lo < hi) {
        int64_t mid = lo + (hi - lo) / 2;
        if (sub[mid] < c) lo = mid + 1; else hi = mid;
    }
    return (lo < n && sub[lo] == c) ? lo : -1;
}

static double subset_in(const void *vctx, int32_t b, int32_t d, int64_t c) {
    subset_ctx *x = (subset_ctx *)vctx;
    int64_t k = subset_index(x->sub, x->n_sub, c);
    if (k < 0) {
        x->missing = 1;
        return NAN;
    }
    return x->I[((int64_t)b * x->nd + d) * x->n_sub + k];
}

void oracle_energy_subset(const oracle_problem *p, int64_t n_sub, const double *I_sub, const double *Tr_sub,
                          double *E_sub) {
    const int32_t nd = p->n_dirs;
    for (int64_t k = 0; k < n_sub; ++k) {
        double e = 0.0;
        for (int32_t b = 0; b < p->n_bands; ++b) {
            double sb = 0.0;
            for (int32_t d = 0; d < nd; ++d) sb += p->w[d] * I_sub[((int64_t)b * nd + d) * n_sub + k];
            e += oracle_weight_at(p, b, Tr_sub ? Tr_sub[k] : NAN) * sb;
        }
        E_sub[k] = e;
    }
}

int oracle_newton_subset(const oracle_problem *p, int64_t n_sub, const double *E_sub, const double *Tr_sub,
                         double *T_sub) {
    double W = 0.0;
    for (int32_t d = 0; d < p->n_dirs; ++d) W += p->w[d];
    int status = ORACLE_OK;
    for (int64_t k = 0; k < n_sub; ++k) {
        int rc = solve_cell(p, W, E_sub[k], Tr_sub ? Tr_sub[k] : NAN, &T_sub[k], NULL);
        if (rc != ORACLE_OK) status = rc;
    }
    return status;
}

int oracle_step_subset(const oracle_problem *p, const int32_t *r, int64_t n_sub, const int64_t *sub,
                       const double *I_sub, const double *T_sub, const double *Tr_sub, int64_t n_sel,
                       const int64_t *sel, double dt, double *Inew_sel, double *T1_sel) {
    const int32_t nb = p->n_bands, nd = p->n_dirs;
    double W = 0.0;
    for (int32_t d = 0; d < nd; ++d) W += p->w[d];
    /* update_one reads T[c] / Tr[c] by global cell id: full-length copies with
     * the subset's values (other entries never read for the selected cells) */
    double *T = (double *)malloc(sizeof(double) * (size_t)p->n_cells);
    double *Tr = (double *)malloc(sizeof(double) * (size_t)p->n_cells);
    if (!T || !Tr) {
        free(T);
        free(Tr);
        return ORACLE_EINVAL;
    }
    for (int64_t k = 0; k < n_sub; ++k) {
        T[sub[k]] = T_sub[k];
        Tr[sub[k]] = Tr_sub ? Tr_sub[k] : NAN;
    }
    int status = ORACLE_OK;
    for (int64_t j = 0; j < n_sel; ++j) {
        subset_ctx ctx = {I_sub, sub, n_sub, nd, 0};
        const int64_t k = sel[j];
        const int64_t c = sub[k];
        double *out = &Inew_sel[j * nb * nd];
        for (int32_t b = 0; b < nb; ++b)
            for (int32_t d = 0; d < nd; ++d)
                out[b * nd + d] = update_one(p, r, T, Tr_sub ? Tr : NULL, subset_in, &ctx, dt, b, d, c);
        if (ctx.missing) {
            status = ORACLE_EINVAL;
            break;
        }
        /* Tr <- T^n, then E and the solve from T^n (oracle_run's order) */
        double e = 0.0;
        for (int32_t b = 0; b < nb; ++b) {
            double sb = 0.0;
            for (int32_t d = 0; d < nd; ++d) sb += p->w[d] * out[b * nd + d];
            e += oracle_weight_at(p, b, T_sub[k]) * sb;
        }
        double Tc = T_sub[k];
        int rc = solve_cell(p, W, e, T_sub[k], &Tc, NULL);
        T1_sel[j] = Tc;
        if (rc != ORACLE_OK) status = rc;
    }
    free(T);
    free(Tr);
    return status;
}
