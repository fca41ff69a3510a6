/*
 * bte.h -- C ABI of the B200-native explicit step of the non-gray phonon
 * Boltzmann transport equation (E. Heisler, S. Mazumder, S. Saurav,
 * A. Deshmukh, H. Sundar, "Automating GPU Scalability for Complex Scientific
 * Models: Phonon Boltzmann Transport Equation", IPDPS 2024).
 *
 * Citations "Lnnn" are lines of the paper text (/root/reference/PAPER.md,
 * not shipped); "SURVEY 8(c) #k" are the readings listed in DESIGN.md.
 *
 * What one step computes (all FP64), for every band-row b, direction d, cell c:
 *
 *   I'[b][d][c] = I + dt ( (I0_b(T_c) - I) / tau_b
 *                          - (v_b / V_c) sum_f A_f (s_d . n_f) I_hat_f )      (Eq. 3, 5)
 *   I_hat_f = I[b][d][c]                if s_d . n_f > 0   (first-order upwind,
 *           = I[b][d][nbr(f)]           interior face       L264-267, L644-647)
 *           = I0_b(T_wall(f))           isothermal wall     (Eq. 6)
 *           = I[b][r_f(d)][c]           symmetric wall, s_r = s_d - 2 (s_d.n_f) n_f
 *   E_c = sum_b c_b sum_d w_d I'[b][d][c]                                     (L412-418)
 *   T_c' solves W sum_b c_b I0_b(T) = E_c  (Newton from T_c, W = sum_d w_d)   (L407-418, L555-561)
 *   I0_b(T) = C_b / expm1(hbar omega_b / (kB T))
 *   c_b = 1/(v_b tau_b) (temp_rule 0, default) or 1/v_b (temp_rule 1)
 *
 * Storage is band-major I[b][d][c] (L777-840: band-parallel loop order) with
 * the cell index fastest.  Band-rows are sharded across ranks (L760-775): rank g
 * of P owns rows [floor(g nb/P), floor((g+1) nb/P)); bands couple only through
 * the per-cell energy, which is summed across ranks once per step (NCCL
 * reduce-scatter of the n_cells partial energies, each rank solves its chunk of
 * cells, all-gather of T: the bytes of one all-reduce).  Cells may be
 * partitioned too (bte_options.cell_part, a halo exchange per step).
 *
 * Conventions for every call:
 *   - All pointers passed IN are borrowed for the duration of the call only and
 *     are HOST pointers unless stated otherwise; inputs are deep-copied.
 *   - Output buffers are caller-allocated HOST memory; getters synchronise the
 *     library's stream before returning.
 *   - Cell order at the ABI is always the caller's order (the library reorders
 *     internally and undoes it in the getters).
 *   - Errors are returned as bte_status; nothing aborts or throws across the
 *     ABI.  bte_last_error() gives the message of the last failure.
 *   - One context per host thread at a time.
 */
#ifndef BTE_H
#define BTE_H

#include <stdint.h>

#if defined(BTE_BUILD) && defined(__GNUC__)
#define BTE_API __attribute__((visibility("default")))
#else
#define BTE_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

typedef struct bte_ctx bte_ctx;     /* opaque; owned by the caller until bte_destroy */
typedef struct bte_group bte_group; /* opaque in-process communicator (bte_group_create) */

typedef enum {
    BTE_OK = 0,
    BTE_EINVAL = 1,  /* invalid argument / input data (message says which) */
    BTE_ENOMEM = 2,  /* device or host allocation failed */
    BTE_ECUDA = 3,   /* CUDA runtime error */
    BTE_ENCCL = 4,   /* NCCL missing or failed */
    BTE_ENOCONV = 5, /* per-cell temperature solve did not converge (E <= 0 or NaN) */
    BTE_ESTATE = 6   /* call not valid in the current state */
} bte_status;

/* Face-based finite-volume mesh (Eq. 3: polygonal/polyhedral cells with m
 * faces of area A_i, L286-292).  2-D meshes are 3-D with unit depth: face areas
 * are edge lengths, volumes are cell areas and every normal has n_z = 0
 * (SURVEY 8(c) #18).  Each cell lists its own faces; an interior face therefore
 * appears once in each of its two cells with opposite normals.
 * Limits: at most 8 faces per cell, n_cells < 2^31. */
typedef struct {
    int32_t dim;                 /* 2 or 3 */
    int64_t n_cells;
    const int64_t *face_offsets; /* [n_cells+1], CSR offsets into the face arrays */
    const int64_t *face_nbr;     /* [n_faces]: >= 0 neighbour cell id;
                                    < 0: boundary face id = -1 - face_nbr */
    const double *face_area;     /* [n_faces], > 0 */
    const double *face_normal;   /* [n_faces][3], unit, outward from the owning cell */
    const double *cell_volume;   /* [n_cells], > 0 */
    const double *cell_centre;   /* [n_cells][3] optional (NULL: keep the caller's order).  A
                                    locality hint only: cells are stored internally in brick
                                    order of these points; results do not depend on it. */
} bte_mesh;

/* Band-rows: one row per (spectral band, polarization) present (L507-514). */
typedef struct {
    int32_t n_bands;
    const double *omega;         /* [n_bands] centre angular frequency, rad/s, > 0 */
    const double *d_omega;       /* [n_bands] width, rad/s (only read when i0_prefactor is NULL) */
    const double *vg;            /* [n_bands] group velocity |v_g|_b, m/s, > 0 */
    const double *tau;           /* [n_bands] relaxation time, s, in (0, +inf]; ignored (may be
                                    NULL) with the rate law below */
    const int32_t *polarization; /* [n_bands] 0 = LA, 1 = TA (only read when i0_prefactor is NULL) */
    const double *i0_prefactor;  /* [n_bands] C_b > 0 of I0_b(T) = C_b / expm1(hbar omega_b / (kB T))
                                    (SURVEY 8(c) #4).  NULL: derived from (omega, d_omega,
                                    polarization) with the built-in quadratic Si dispersion
                                    omega = v_s k + c k^2 (LA 9.01e3 m/s, -2.0e-7 m^2/s; TA 5.23e3,
                                    -2.26e-7) as C_b = hbar omega k^2 d_omega / (8 pi^3);
                                    d_omega and polarization are then required (EINVAL otherwise,
                                    or if omega lies above the branch maximum) */
    /* Optional temperature-dependent relaxation times (the paper
     * keeps tau as a per-cell variable that depends on T, L666-669, `beta` per
     * cell L1352-1353).  NULL rate_a: constant tau.  Else, per band-row and cell,
     *     1/tau_b(T) = rate_a[b] + rate_b[b] T exp(-rate_theta[b] / T)   (1/s)
     * with all three arrays >= 0 and finite.  The rates of step n are those of
     * the cell temperature of step n-1 (reading 22): the relaxation
     * of a step and the R2 weights 1/(v tau) of the temperature solve that
     * ends the previous step use the same rates, so the RTA energy balance is
     * exact.  The library keeps that rate temperature per cell: t_init at
     * bte_create, T at bte_set_equilibrium, T^n after step n. */
    const double *rate_a, *rate_b, *rate_theta;
} bte_bands;

/* Discrete directions (L514-518, L654-664): unit vectors and solid-angle weights. */
typedef struct {
    int32_t n_dirs;
    const double *s; /* [n_dirs][3], unit */
    const double *w; /* [n_dirs], > 0 */
} bte_dirs;

/* Boundary conditions per boundary face id (Eq. 6). */
#define BTE_BC_ISOTHERMAL 0
#define BTE_BC_SYMMETRY 1
typedef struct {
    int64_t n_bfaces;
    const int32_t *kind;  /* [n_bfaces] BTE_BC_ISOTHERMAL or BTE_BC_SYMMETRY */
    const double *t_wall; /* [n_bfaces] wall temperature (K, > 0) of isothermal faces */
} bte_bcs;

/* bte_options.flags */
#define BTE_FLAG_PROFILE 1u       /* record CUDA events around every phase (see bte_stats) */
#define BTE_FLAG_GENERIC_FACES 2u /* never use the opposite-face-pair layout (testing) */
#define BTE_FLAG_NO_TMA 4u        /* register-pipelined generic-face flux kernel instead of the
                                     TMA-staged ones (testing / comparison) */
/* (8u was an opt-in stencil-window kernel, removed: L2-bound) */
#define BTE_FLAG_NO_BOX 16u       /* structured 2-D / 3-D box grids: do not use the box kernel
                                     (tensor-copy z-marching tiles, the default there) */

typedef struct {
    double t_init;            /* IC: T = t_init, I = I0_b(t_init) (L585-588, L678-684) */
    int32_t temp_rule;        /* 0: R2, c_b = 1/(v_b tau_b) (default); 1: R1, c_b = 1/v_b (the
                                 energy-equivalent temperature); 2: R3, one linearised
                                 "first-law" step T + dE / C(T) with the R1 weights per step
                                 (L413-415; reading 5) */
    double newton_rtol;       /* temperature solve tolerance (default 1e-12; L555-561): an
                                 iterate T is accepted once its Newton correction
                                 |g/g'| <= max(rtol/100, 16 eps) T, i.e. within ~rtol/100
                                 of the root the oracle's |dT| <= rtol T test converges to
                                 (reading 25); the bisection bracket to rtol T */
    int32_t newton_max_iter;  /* default 50 (evaluations); bisection fallback after that */
    int32_t rank, world;      /* band sharding; world == 1: single GPU, no NCCL */
    int32_t device;           /* CUDA device ordinal */
    const void *nccl_unique_id; /* world > 1: 128-byte ncclUniqueId from bte_nccl_unique_id()
                                   on rank 0, broadcast by the caller.  NULL with world > 1:
                                   no communicator; the caller reduces the energy itself
                                   through the split-step calls (bte_step returns ESTATE).
                                   An id with world == 1 builds a one-rank communicator and
                                   runs the all-reduce path (testing) */
    void *stream;             /* cudaStream_t to launch on (NULL: library-owned stream) */
    uint32_t flags;           /* BTE_FLAG_* */
    int32_t max_spare_slabs;  /* band slabs of workspace: <= 0 auto (double buffer when it
                                 fits, else slab rotation), k > 0 forces at most k */
    int32_t block_threads;    /* 0 auto; else 64..1024, multiple of 32 */
    int32_t band_group;       /* 0 auto; else 1..8 band-rows per thread (box kernel: band-rows
                                 per thread block, any >= 1) */
    int32_t dir_chunk;        /* 0 auto; else directions per thread block (box kernel: rounded
                                 down to whole 4-direction orbits) */
    /* Cell partitioning (the paper's cell-parallel split with a
     * Metis-style partition, L728-735, L768-772, Fig. 3-4), optionally combined
     * with band sharding.  NULL cell_part: none (band sharding only).  Else
     * every rank passes the WHOLE mesh and the same partition; rank r owns the
     * cells of part r % n_cell_parts and the band-rows of band group
     * r / n_cell_parts (world / n_cell_parts groups, rows split as above).
     * Every step first exchanges, with the ranks of the same band group, the
     * old-level intensities its cut faces read (halo; only the directions that
     * flow across the cut), then runs the same step on the owned cells; the
     * energy is reduced over the ranks of the same part.  All cell-indexed
     * arrays at the ABI (T, E, I) then hold the OWNED cells in ascending global
     * id (bte_local_cells).  Without a communicator the caller moves the halo
     * with bte_halo_export / bte_halo_import before bte_step_begin. */
    const int32_t *cell_part; /* [n_cells] part id in [0, n_cell_parts) */
    int32_t n_cell_parts;     /* >= 1; world must be a multiple of it */
    /* In-process communicator instead of NCCL (bte_group_create): the `world`
     * ranks are host threads of this process, rank r calling every collective
     * entry point from its own thread, each context on any device (several may
     * share one).  The per-step exchanges (reduce-scatter / all-gather of the
     * energy and T, the all-reduce variants, the halo send / receive group, the
     * band-group split) then run as stream-ordered device copies between the
     * ranks' buffers with the same semantics as the NCCL calls; no CUDA graphs.
     * NULL: NCCL (nccl_unique_id) or no communicator.  EINVAL if the group's
     * size differs from world or an NCCL id is passed too. */
    bte_group *group;
    /* Temperature-dependent relaxation times only: 0 (default) the rates of a
     * step are those of the previous step's temperature (DESIGN.md reading
     * 22: the R2 weights of the solve that produced T^n and the relaxation of
     * step n use the same rates, so the RTA energy balance is exact); 1 the
     * literal post-step refresh of the Finch loop (L707-716: I0 and tau both
     * from the new T), step n relaxes with tau(T^n) (reading 26). */
    int32_t rates_now;
} bte_options;

/* Per-context counters since creation / the last bte_reset_stats. Phase
 * times need BTE_FLAG_PROFILE and are sums of CUDA-event intervals on the
 * library stream. */
typedef struct {
    int64_t steps;
    int64_t kernel_launches;   /* kernels launched by bte_step */
    int64_t updates;           /* (cell, dir, band) unknowns advanced on this rank */
    double ms_flux_interior;   /* interior-cell flux + relaxation + energy partial */
    double ms_flux_boundary;   /* boundary-cell kernel */
    double ms_allreduce;       /* slot reduce + NCCL energy exchange (world > 1) */
    double ms_newton;          /* temperature solve + I0 refresh */
    double ms_total;           /* first to last event of the profiled steps */
    int32_t newton_iter_max;   /* max Newton iterations of any cell */
    int32_t spare_slabs;       /* workspace band slabs in use */
    int32_t n_interior_cells;
    int32_t band_group;
    int32_t block_threads;
    int32_t dir_chunks;        /* direction chunks per launch (grid.y factor) */
    int32_t flux_variant;      /* flux kernel in use: 0 register-pipelined generic faces,
                                  3 TMA-staged opposite-face pairs, 4 ... + uniform geometry,
                                  6 box (structured 2-D / 3-D grid, tensor copies), 7
                                  TMA-staged generic faces (unstructured meshes) */
    double ms_halo;            /* cell partitioning: halo pack + exchange + unpack */
    int64_t halo_bytes;        /* halo bytes this rank sends per step (all segments) */
    int64_t flux_launches;     /* flux-kernel launches (a1-a3), part of kernel_launches */
    int64_t graph_replays;     /* 2-step CUDA-graph replays inside bte_step (their kernels are
                                  counted in kernel_launches) */
} bte_stats;

/* Fill *o with the defaults (t_init 300, temp_rule 0, rtol 1e-12, 50 iters,
 * rank 0 / world 1 / device 0, everything else 0/NULL).  Newton controls:
 * SURVEY 8(c) #6 (the paper gives none).  EINVAL if o is NULL. */
BTE_API bte_status bte_options_default(bte_options *o);

/* In-process communicator of `world` ranks (see bte_options.group).  *out is
 * owned by the caller; destroy it after every context that uses it.  EINVAL
 * if world < 1 or out is NULL. */
BTE_API bte_status bte_group_create(int32_t world, bte_group **out);
BTE_API void bte_group_destroy(bte_group *g);

/* The problem statement of the paper (mesh + FVM, L286-292, L719-722; band
 * table with omega, v_g, tau, polarization, L507-514, L1339-1359; direction
 * set, L514-518, L654-664; isothermal / symmetric BCs, L563-607): validate and
 * deep-copy it, build the device layout (face slots, reflection maps,
 * isothermal ghost tables, slab pool) and initialise the state to the
 * equilibrium IC I = I0_b(t_init), T = t_init (L585-588, L678-684).
 * All pointers are host pointers borrowed for the call; *out is owned by the
 * caller (bte_destroy).  Collective when world > 1 with a communicator.
 * EINVAL on: dim not 2/3; non-positive V, A, w, C, omega, v or tau; non-unit
 * normals or directions; n_z != 0 in 2-D; a face id out of range; > 8 faces in
 * a cell; a symmetric wall whose reflected direction is not in the set (1e-10);
 * all temperature weights zero; more than 128 band-rows on one rank or 1024 in
 * all.  ENOMEM if the state does not fit the device; ECUDA / ENCCL on runtime
 * or communicator failures.  On error *out is NULL and bte_last_error(NULL)
 * says why. */
BTE_API bte_status bte_create(const bte_mesh *mesh, const bte_bands *bands, const bte_dirs *dirs,
                      const bte_bcs *bcs, const bte_options *opts, bte_ctx **out);

/* n explicit steps of size dt: forward Euler on the finite-volume form (Eq.
 * 2-3, L269-292) of the phonon BTE (Eq. 4-5) with first-order upwind
 * face values (L264-267, L644-647), the Eq. 6 ghosts (L563-607), the per-cell
 * energy (L412-418) summed across ranks (L760-766) and the temperature solve
 * that refreshes I0 (L407-418, L555-561, L707-716).  Collective when world > 1;
 * returns after the steps completed (host-synchronous).
 * EINVAL if dt <= 0 or dt exceeds the positivity bound
 * 1 / max_{c,b,d} (1/tau_b + v_b sum_f (A_f/V_c) max(s_d.n_f, 0)) (see
 * bte_dt_bound); ESTATE inside a split step or with world > 1
 * and no communicator.  ENOCONV if a cell's temperature solve failed
 * (E <= 0 or non-finite): stepping stops at that step, the state is the one at
 * its end (the failed cells keep their previous T), the remaining steps are not
 * taken, and bte_get_stats().steps counts the steps taken.  With cell
 * partitioning the failure is reported by the ranks owning the failed cells. */
BTE_API bte_status bte_step(bte_ctx *ctx, double dt, int64_t n);

/* Largest admissible dt (the positivity bound above, over all bands; with the
 * rate law, rates at the highest temperature the state can reach: the max of
 * t_init, the wall temperatures and the last set / solved T, P10).  Host
 * pointer out.  EINVAL on NULL. */
BTE_API bte_status bte_dt_bound(const bte_ctx *ctx, double *dt_max);

/* Temperature of the CURRENT state under `rule` (0 R2, 1 R1 energy-equivalent,
 * 2 R3 one linearised "first law" step from the current T, L413-415), without
 * changing the state:
 * energy reduction with that rule's weights, all-reduce (collective when
 * world > 1), Newton from the current T.  T[n_cells] host, caller order.
 * the paper's temperature relation is under-specified
 * (L413-418), so the other readings are offered as outputs.  ENOCONV if a
 * cell's solve fails; ESTATE with world > 1 and no communicator. */
BTE_API bte_status bte_get_temperature_rule(const bte_ctx *ctx, int32_t rule, double *T);

/* The lattice temperature T_c of the current state, the output of the
 * per-cell solve (L407-418, L555-561; Fig. 6 "temperature"), into the
 * caller's host buffer T[n_cells] in caller cell order (owned cells under cell
 * partitioning).  Replicated on every rank.  Synchronises the library stream.
 * EINVAL on NULL; ECUDA on a runtime failure. */
BTE_API bte_status bte_get_temperature(const bte_ctx *ctx, double *T);

/* The intensity field I[b][d][c] of the current state (the unknowns of Eq. 5,
 * L546-553; band-major storage, L777-840) for global band-rows [b_lo, b_hi),
 * which must lie inside this rank's bte_band_range, into the caller's host
 * buffer I[b_hi-b_lo][n_dirs][n_cells] (caller cell order).  Synchronises the
 * library stream.  EINVAL for rows outside the range or NULL; ESTATE inside a
 * split step. */
BTE_API bte_status bte_get_intensity(const bte_ctx *ctx, int32_t b_lo, int32_t b_hi, double *I);

/* Overwrite rows [b_lo, b_hi) of I from the caller's host buffer (layout of
 * bte_get_intensity; restart / checkpoint of the explicit state, L398-404
 * "u = u_new").  T is NOT changed; call bte_solve_temperature after the last
 * row is set.  Errors as bte_get_intensity. */
BTE_API bte_status bte_set_intensity(bte_ctx *ctx, int32_t b_lo, int32_t b_hi, const double *I);

/* T <- temperature of the current I: the energy integral over all directions
 * and bands (L412-418), summed across ranks (L760-766), the per-cell Newton
 * solve from the current T (L555-561), and I0 refreshed
 * (L707-716).  Collective when world > 1.  ENOCONV if a cell's solve fails
 * (its T is kept); ESTATE inside a split step or world > 1 without a
 * communicator. */
BTE_API bte_status bte_solve_temperature(bte_ctx *ctx);

/* Set T (host buffer, caller order) and I = I0_b(T_c) for every local row
 * (local thermal equilibrium, the IC of L585-588, L678-684).  Not collective.
 * EINVAL if some T_c <= 0 or non-finite; ESTATE inside a split step. */
BTE_API bte_status bte_set_equilibrium(bte_ctx *ctx, const double *T);

/* This rank's band-rows [b_lo, b_hi) (band-parallel split, L773-775:
 * [floor(g nb / G), floor((g+1) nb / G)) for band group g of G).  EINVAL on NULL. */
BTE_API bte_status bte_band_range(const bte_ctx *ctx, int32_t *b_lo, int32_t *b_hi);

/* Split step, for callers that reduce the energy themselves (the band
 * coupling of L760-766 done outside the library): begin = flux / relaxation
 * of the local rows (Eq. 3, 5, 6) and the local energy partial (L412-418);
 * get / set energy move E[n_cells] (host buffer, caller order); finish =
 * temperature solve from the set energy, I0 refresh and state advance.
 * bte_step(ctx, dt, 1) == begin; (reduce E); finish.  ESTATE for begin twice
 * or finish without begin; EINVAL for dt as bte_step; ENOCONV from finish as
 * bte_step. */
BTE_API bte_status bte_step_begin(bte_ctx *ctx, double dt);
BTE_API bte_status bte_get_energy(const bte_ctx *ctx, double *E);
BTE_API bte_status bte_set_energy(bte_ctx *ctx, const double *E);
BTE_API bte_status bte_step_finish(bte_ctx *ctx);

/* Cell partitioning (see bte_options.cell_part; the paper's cell-parallel
 * split, L728-735, L768-772).  Owned cells of this rank: *n_local, and (ids !=
 * NULL) their global ids ascending into the caller's host buffer ids[*n_local].
 * Without partitioning: all cells, ids 0..n_cells-1.  EINVAL on NULL ctx / n_local. */
BTE_API bte_status bte_local_cells(const bte_ctx *ctx, int64_t *n_local, int64_t *ids);

/* Halo segment sizes with part `part` (doubles): *n_send = values this rank
 * sends to it, *n_recv = values it receives from it (0 and 0 if the parts share
 * no face or part is this rank's own).  Segment layout [k][j][i]: local band-row
 * k, the segment's directions j (ascending ids d with s_d . n_f < 0 at the
 * reading cell's cut face f), the segment's cells i (ascending global id of
 * the writing part's cells that cut faces of the reading part point to). */
BTE_API bte_status bte_halo_size(const bte_ctx *ctx, int32_t part, int64_t *n_send, int64_t *n_recv);

/* Caller-driven halo exchange (no communicator, e.g. partitions emulated on one
 * device): export writes the current I^n values this rank sends to `part` into
 * buf[n_send] (host); import stores the values received from `part`
 * (buf[n_recv], host) as this rank's halo.  Call import for every neighbour
 * part before bte_step_begin; the halo is read by the next flux only.  EINVAL
 * for a part out of range, ESTATE inside a split step. */
BTE_API bte_status bte_halo_export(const bte_ctx *ctx, int32_t part, double *buf);
BTE_API bte_status bte_halo_import(bte_ctx *ctx, int32_t part, const double *buf);

/* Counters (see bte_stats) into the caller's struct / reset them (the
 * paper's per-phase timing of Figs. 5 and 8, L854-857, L871-873).  EINVAL on NULL. */
BTE_API bte_status bte_get_stats(const bte_ctx *ctx, bte_stats *st);
BTE_API bte_status bte_reset_stats(bte_ctx *ctx);

/* 128-byte NCCL unique id into the caller's buffer (call on rank 0 only, then
 * broadcast; the multi-GPU band sharding of L760-775).  ENCCL if the NCCL
 * library cannot be loaded (BTE_NCCL_LIB overrides the search); EINVAL on NULL. */
BTE_API bte_status bte_nccl_unique_id(void *id128);

/* Message of the last failure on ctx (ctx may be NULL: last bte_create /
 * global failure of this thread).  Never NULL; owned by the library, valid
 * until the next call on ctx. */
BTE_API const char *bte_last_error(const bte_ctx *ctx);
BTE_API const char *bte_status_string(bte_status s);

/* Release the context: device memory, the library-owned stream, the NCCL
 * communicator / group endpoint (synchronises first).  Not collective.  NULL
 * is a no-op.  Every pointer obtained from ctx is invalid afterwards. */
BTE_API void bte_destroy(bte_ctx *ctx);

#ifdef __cplusplus
}
#endif
#endif /* BTE_H */
