/*
 * bte_oracle.h -- CPU ORACLE for the non-gray phonon BTE explicit step.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this library.  It
 * shares no code, header, table or constant with the CUDA path under
 * paper_conf_ipps_heislersdms24_b200/csrc, and it never takes an input from it.
 *
 * It is a plain, slow, obviously-correct transcription of the method of
 * E. Heisler et al., IPDPS 2024 ("PAPER", /root/reference/PAPER.md):
 *   Eq. 2-3   forward Euler + cell-average quadrature     (L269-292)
 *   upwind    conditional(b.n > 0, CELL1_u, CELL2_u)       (L264-267, L644-647)
 *   Eq. 5     FVM BTE per (d, b) with RTA source           (L529-553)
 *   Eq. 6     isothermal / symmetric ghost intensities     (L563-576, L602-607)
 *   T update  energy over all (d, b) per cell + nonlinear  (L407-418, L555-561,
 *             temperature recovery each step                L707-716)
 * with the readings of SURVEY.md 8(c) (listed in DESIGN.md 3).
 *
 * Layouts: I[b][d][c] (cell fastest, user cell order); T[c]; mesh in CSR face
 * lists (face_nbr >= 0 neighbour, < 0 => boundary face id -1 - face_nbr).
 * All floating point is IEEE double, summed in ascending stored order.
 */
#ifndef BTE_ORACLE_H
#define BTE_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct {
    /* mesh */
    int32_t dim;
    int64_t n_cells;
    const int64_t *face_offsets; /* [n_cells+1] */
    const int64_t *face_nbr;     /* [n_faces] */
    const double *face_area;     /* [n_faces] */
    const double *face_normal;   /* [n_faces][3] outward unit normal */
    const double *cell_volume;   /* [n_cells] */
    /* band-rows */
    int32_t n_bands;
    const double *omega; /* rad/s */
    const double *vg;    /* m/s */
    const double *tau;   /* s, +inf allowed */
    const double *C;     /* I0_b(T) = C_b / expm1(hbar omega_b / (kB T)) */
    /* directions */
    int32_t n_dirs;
    const double *s; /* [n_dirs][3] */
    const double *w; /* [n_dirs] */
    /* boundary faces */
    int64_t n_bfaces;
    const int32_t *bkind;  /* 0 isothermal, 1 symmetric */
    const double *t_wall;  /* K, isothermal faces */
    /* temperature rule and Newton controls */
    int32_t temp_rule;     /* 0: c_b = 1/(v_b tau_b) (R2), 1: c_b = 1/v_b (R1), 2: R3 = one
                              linearised first-law step dT = dE / C(T) with the R1 weights
                              (L413-415 "can be approximated ... using the first law";
                              SURVEY 8(c) #5, 8(f) N4) */
    double newton_rtol;    /* stop when |dT| <= rtol T */
    int32_t newton_maxit;
    /* Temperature-dependent relaxation times ("tau ... dependent
     * on temperature ... mutable values for each cell", L666-669, beta[b] per
     * cell L1352-1353).  NULL rate_a: constant tau above.  Else
     *   1/tau_b(T) = rate_a[b] + rate_b[b] T exp(-rate_theta[b] / T)
     * evaluated per cell at the rate temperature Tr (reading 22:
     * the rates of step n are those of the temperature of step n-1, so the
     * R2 temperature equation and the relaxation use the same rates). */
    const double *rate_a, *rate_b, *rate_theta;
    /* 0 (default): the rates lag one step (reading 22: step n relaxes with
     * tau(T^{n-1}), its temperature solve weighs with tau(T^n)).  1: the
     * literal post-step refresh of the Finch loop (L707-716): I0 and tau are
     * both refreshed from the new T, so step n relaxes with tau(T^n) and its
     * solve weighs with tau(T^n) too (Tr = T at the start of every step;
     * DESIGN.md reading 26). */
    int32_t rates_now;
} oracle_problem;

/* return codes */
#define ORACLE_OK 0
#define ORACLE_EINVAL 1
#define ORACLE_ENOCONV 5

/* I0_b(T) = C / expm1(theta/T), theta = hbar omega / kB. */
double oracle_I0(double C, double omega, double T);
/* c_b, the temperature weight of band-row b under temp_rule (constant rates). */
double oracle_weight(const oracle_problem *p, int32_t b);
/* 1/tau_b at rate temperature Tr (the law, or the constant 1/tau_b; +inf -> 0). */
double oracle_rate(const oracle_problem *p, int32_t b, double Tr);
/* c_b at rate temperature Tr: R2 rate/v_b, R1 1/v_b. */
double oracle_weight_at(const oracle_problem *p, int32_t b, double Tr);

/* Specular map (Eq. 6): r[f][d] = d' with s_d' = s_d - 2 (s_d.n_f) n_f within
 * 1e-10, for every symmetric boundary face f; -1 for isothermal faces.
 * r is [n_bfaces][n_dirs].  Returns ORACLE_EINVAL if a reflection is missing. */
int oracle_reflection_map(const oracle_problem *p, int32_t *r);

/* Intensity update of Eq. 3/5 with the Eq. 6 ghosts for band-rows [b_lo, b_hi):
 * Inew = I + dt ((I0_b(T_c) - I)/tau_b - (v_b/V_c) sum_f A_f (s_d.n_f) I_hat_f),
 * 1/tau_b = oracle_rate(p, b, Tr_c) (Tr may be NULL with constant rates). */
void oracle_update_intensity(const oracle_problem *p, const int32_t *r, const double *T, const double *Tr,
                             const double *I, double *Inew, double dt, int32_t b_lo, int32_t b_hi);

/* E_c = sum_{b in [b_lo,b_hi)} c_b(Tr_c) sum_d w_d I[b][d][c]  (L412-418). E is
 * overwritten (not accumulated).  Tr may be NULL with constant rates. */
void oracle_energy(const oracle_problem *p, const double *I, const double *Tr, int32_t b_lo, int32_t b_hi,
                   double *E);

/* Per-cell temperature: solve W sum_b c_b(Tr_c) I0_b(T) = E_c by Newton from
 * T_c (bisection safeguard).  T is in/out; iters (may be NULL) gets the
 * per-cell Newton iteration count.  Returns ORACLE_ENOCONV if any cell fails. */
int oracle_newton(const oracle_problem *p, const double *E, const double *Tr, double *T, int32_t *iters);

/* Equilibrium field: I[b-b_lo][d][c] = I0_b(T_c) for b in [b_lo, b_hi) (the IC
 * "equilibrium intensity for a uniform temperature", L678-684). */
void oracle_equilibrium(const oracle_problem *p, const double *T, int32_t b_lo, int32_t b_hi, double *I);

/* Whole explicit steps: I (all bands), T and the rate temperature Tr in/out
 * (Tr may be NULL with constant rates).  Per step: (rates_now: Tr <- T;)
 * Inew from (I, T, Tr); Tr <- T; E and the Newton solve with the weights at
 * the new Tr; I <- Inew.
 * Returns 0 or an error. */
int oracle_run(const oracle_problem *p, double dt, int64_t nsteps, double *I, double *T, double *Tr);

/* One step at selected cells when I^n is the equilibrium of the temperature
 * field T0 (I^n[b][d][c] = I0_b(T0_c)) and the rate temperature is T0 too.
 * Writes Inew_sel[k][b][d] and the Newton temperature T1_sel[k] of cell
 * cells[k] (initial guess T0).  Used for sampled checks at sizes where the
 * full field does not fit on the host. */
int oracle_step_cells_equilibrium(const oracle_problem *p, const int32_t *r, const double *T0,
                                  const int64_t *cells, int64_t n_sel, double dt,
                                  double *Inew_sel, double *T1_sel);

/* The same on a SUBSET of cells whose intensities are given explicitly (full
 * fields that do not fit on the host, with a direction-dependent state).
 * sub[n_sub]: ascending cell ids; I_sub[b][d][k] the intensity of cell sub[k].
 *   oracle_energy_subset: E_sub[k] = E of cell sub[k] (weights at Tr_sub[k]).
 *   oracle_newton_subset: T_sub in/out, the per-cell solve of oracle_newton.
 *   oracle_step_subset:   one explicit step of the cells sub[sel[j]] (their
 *     face neighbours must be in sub): Inew_sel[j][b][d] from (I_sub, T_sub,
 *     Tr_sub), then E and the solve with the weights at T_sub (Tr <- T^n, as
 *     in oracle_run) from T_sub: T1_sel[j].
 * ORACLE_EINVAL if a neighbour is missing from sub; ORACLE_ENOCONV as above. */
void oracle_energy_subset(const oracle_problem *p, int64_t n_sub, const double *I_sub, const double *Tr_sub,
                          double *E_sub);
int oracle_newton_subset(const oracle_problem *p, int64_t n_sub, const double *E_sub, const double *Tr_sub,
                         double *T_sub);
int oracle_step_subset(const oracle_problem *p, const int32_t *r, int64_t n_sub, const int64_t *sub,
                       const double *I_sub, const double *T_sub, const double *Tr_sub, int64_t n_sel,
                       const int64_t *sel, double dt, double *Inew_sel, double *T1_sel);

#ifdef __cplusplus
}
#endif
#endif
