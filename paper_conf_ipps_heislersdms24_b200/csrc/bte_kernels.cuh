// bte_kernels.cuh -- sm_100a kernels of the explicit phonon-BTE step.
//
// Paper: E. Heisler et al., IPDPS 2024; "Lnnn" = line of PAPER.md.
//
//   flux_kernel    Eq. 3 / Eq. 5 forward-Euler update with the first-order
//                  upwind face flux (L264-292, L529-553, L644-647), the RTA
//                  source (I0 - I)/tau, the Eq. 6 ghosts on boundary cells
//                  (L563-607) and the fused per-cell energy partial
//                  sum_b c_b sum_d w_d I' (L412-418).  HBM-bound: 16 B per
//                  (cell, dir, band) update (read I^n, write I^{n+1}).
//   newton_kernel  per-cell temperature from the energy (L407-418, L555-561,
//                  L707-716) and the I0 table of the next step.
//   small kernels  reductions, gathers/scatters into caller cell order,
//                  equilibrium initialisation, isothermal ghost table, dt bound.
//
// Layout: I slab of band-row b = [n_dirs][n_cells] doubles in a
// slab pool; cells reordered interior-first; per-cell face geometry stored as
// padded face slots j < MF in struct-of-arrays form [j][cell]:
//   nbr[j][c] (int32), g[j][c] = (A_f / V_c) n_f (FP64, DIM components),
//   and for boundary cells kind[j][c] (0 interior, 1 isothermal, 2 symmetric)
//   and aux[j][c] (isothermal ghost column / reflection-class row).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace bte {

constexpr int kMaxBandsPerLaunch = 128;
constexpr int kMaxThreads = 256;

enum : int8_t { kFaceInterior = 0, kFaceIso = 1, kFaceSym = 2 };

struct FluxParams {
    int32_t nc;          // cells = plane stride
    int32_t cell_begin;  // cell range of this launch (internal order)
    int32_t cell_end;
    int32_t nd;          // directions
    int32_t dchunk;      // directions per block
    int32_t n_dchunks;
    int32_t nbl;         // band-rows in this launch
    int32_t bg;          // band-rows per thread group (<= BG)
    int32_t band0;       // rank-local index of the launch's first band-row
    int32_t slot0;       // first energy-partial slot of this launch
    int64_t slab_elems;  // nd * nc
    double *pool;        // slab pool
    const double *i0;    // [nb_loc][nc]  I0_b(T_c) of the current step
    double *part;        // [n_slots][nc] energy partials
    const int32_t *nbr;  // [MF][nc]
    const double *gx, *gy, *gz;  // [MF][nc]
    const int8_t *kind;  // [MF][nc] (boundary cells only are read)
    const int32_t *aux;  // [MF][nc]
    const int32_t *refl; // [n_refl_classes][nd]
    const double *i0w;   // [nb_loc][n_iso]  I0_b(T_wall) per isothermal face
    int32_t n_iso;
    const double4 *dirs; // [nd] {s_x, s_y, s_z, w}
    const double *inv_tau, *vg, *cw;  // [nb_loc]
    double dt;
    int32_t in_slot[kMaxBandsPerLaunch];
    int32_t out_slot[kMaxBandsPerLaunch];
};

// One thread owns one cell and a (band group, direction chunk) of its unknowns.
// Per direction it forms alpha_j = s_d . g_j for its faces once and reuses it for
// every band-row of the group; per band-row it streams I^n[b][d][c] in, reads the
// upwind neighbours of the inflow faces (L1/L2 hits: same plane), and streams
// I^{n+1} out.  The energy partial stays in registers until the end.
template <int DIM, int MF, int BG, bool BND>
__global__ void __launch_bounds__(kMaxThreads)
flux_kernel(const __grid_constant__ FluxParams p) {
    const int c = p.cell_begin + blockIdx.x * blockDim.x + threadIdx.x;
    if (c >= p.cell_end) return;
    const int grp = blockIdx.y / p.n_dchunks;
    const int dch = blockIdx.y - grp * p.n_dchunks;
    const int lg0 = grp * p.bg;  // launch-local first band-row of the group
    const int nbg = min(p.bg, p.nbl - lg0);
    const int d0 = dch * p.dchunk;
    const int d1 = min(p.nd, d0 + p.dchunk);
    const int nc = p.nc;

    int nbr[MF];
    double gx[MF], gy[MF], gz[MF];
    int8_t kind[MF];
    int aux[MF];
#pragma unroll
    for (int j = 0; j < MF; ++j) {
        nbr[j] = __ldg(p.nbr + (size_t)j * nc + c);
        gx[j] = __ldg(p.gx + (size_t)j * nc + c);
        gy[j] = __ldg(p.gy + (size_t)j * nc + c);
        gz[j] = DIM == 3 ? __ldg(p.gz + (size_t)j * nc + c) : 0.0;
        if (BND) {
            kind[j] = p.kind[(size_t)j * nc + c];
            aux[j] = __ldg(p.aux + (size_t)j * nc + c);
        }
    }

    const double *inb[BG];
    double *outb[BG];
    double src[BG], diag[BG], kv[BG], acc[BG];
    int lb[BG];
#pragma unroll
    for (int k = 0; k < BG; ++k) {
        const int kk = k < nbg ? k : 0;
        lb[k] = p.band0 + lg0 + kk;
        inb[k] = p.pool + (int64_t)p.in_slot[lg0 + kk] * p.slab_elems;
        outb[k] = p.pool + (int64_t)p.out_slot[lg0 + kk] * p.slab_elems;
        const double dtit = p.dt * __ldg(p.inv_tau + lb[k]);
        src[k] = dtit * __ldg(p.i0 + (size_t)lb[k] * nc + c);  // dt/tau I0_b(T_c)
        diag[k] = 1.0 - dtit;
        kv[k] = p.dt * __ldg(p.vg + lb[k]);
        acc[k] = 0.0;
    }

    for (int d = d0; d < d1; ++d) {
        const double2 sxy = __ldg(reinterpret_cast<const double2 *>(p.dirs + d));
        const double2 szw = __ldg(reinterpret_cast<const double2 *>(p.dirs + d) + 1);
        const double4 sd = make_double4(sxy.x, sxy.y, szw.x, szw.y);
        double a[MF];
        double out = 0.0;
#pragma unroll
        for (int j = 0; j < MF; ++j) {
            a[j] = DIM == 3 ? fma(sd.z, gz[j], fma(sd.y, gy[j], sd.x * gx[j]))
                            : fma(sd.y, gy[j], sd.x * gx[j]);
            out += fmax(a[j], 0.0);  // outflow faces use the cell's own value
        }
        const size_t po = (size_t)d * nc;
#pragma unroll
        for (int k = 0; k < BG; ++k) {
            if (k < nbg) {
                const double *pl = inb[k] + po;
                const double ic = __ldg(pl + c);
                double infl = 0.0;
#pragma unroll
                for (int j = 0; j < MF; ++j) {
                    if (a[j] < 0.0) {  // inflow: upwind neighbour or ghost
                        double v;
                        if (!BND || kind[j] == kFaceInterior) {
                            v = __ldg(pl + nbr[j]);
                        } else if (kind[j] == kFaceIso) {
                            v = __ldg(p.i0w + (size_t)lb[k] * p.n_iso + aux[j]);
                        } else {  // specular: reflected direction, same cell, old level
                            const int r = __ldg(p.refl + (size_t)aux[j] * p.nd + d);
                            v = __ldg(inb[k] + (size_t)r * nc + c);
                        }
                        infl = fma(a[j], v, infl);
                    }
                }
                // I' = I (1 - dt/tau - dt v out) + dt/tau I0 - dt v sum_in alpha I_nbr
                const double inew = fma(ic, diag[k] - kv[k] * out, fma(-kv[k], infl, src[k]));
                __stcs(outb[k] + po + c, inew);
                acc[k] = fma(sd.w, inew, acc[k]);
            }
        }
    }
    double e = 0.0;
#pragma unroll
    for (int k = 0; k < BG; ++k)
        if (k < nbg) e = fma(__ldg(p.cw + lb[k]), acc[k], e);
    p.part[(size_t)(p.slot0 + grp * p.n_dchunks + dch) * nc + c] = e;
}

// ---------------------------------------------------------------- temperature

struct NewtonParams {
    int32_t nc;
    int32_t nb;            // all band-rows (global)
    int32_t n_slots;       // energy partial slots (when E == nullptr)
    const double *part;
    const double *E;       // reduced energy, or nullptr to sum the slots
    double *T;
    double *i0;            // [nb_loc][nc] written for global rows [b_lo, b_lo + nb_loc)
    int32_t b_lo, nb_loc;
    const double *Cb, *theta, *cw;  // [nb] global
    double W, rtol;
    int32_t maxit;
    int32_t *iter_max;
    int32_t *fail;
};

struct Gsum { double g, gp; };

// g(T) = W sum_b c_b I0_b(T) - E and g'(T), I0 = C / expm1(theta/T),
// I0' = I0 (x/T) (1 + 1/expm1(x)), x = theta/T.
__device__ __forceinline__ Gsum g_eval(const double *sC, const double *sTh, const double *sW,
                                       int nb, double W, double E, double T) {
    double g = 0.0, gp = 0.0;
    const double it = 1.0 / T;
    for (int b = 0; b < nb; ++b) {
        const double x = sTh[b] * it;
        const double em1 = expm1(x);
        const double i0 = sC[b] / em1;
        g = fma(sW[b], i0, g);
        gp = fma(sW[b], i0 * (x * it) * (1.0 + 1.0 / em1), gp);
    }
    return {W * g - E, W * gp};
}

__device__ __forceinline__ double g_only(const double *sC, const double *sTh, const double *sW,
                                         int nb, double W, double E, double T) {
    double g = 0.0;
    for (int b = 0; b < nb; ++b) g = fma(sW[b], sC[b] / expm1(sTh[b] / T), g);
    return W * g - E;
}

__global__ void newton_kernel(const __grid_constant__ NewtonParams p) {
    extern __shared__ double sm[];
    double *sC = sm, *sTh = sm + p.nb, *sW = sm + 2 * p.nb;
    for (int b = threadIdx.x; b < p.nb; b += blockDim.x) {
        sC[b] = p.Cb[b];
        sTh[b] = p.theta[b];
        sW[b] = p.cw[b];
    }
    __syncthreads();
    const int c = blockIdx.x * blockDim.x + threadIdx.x;
    if (c >= p.nc) return;
    double E;
    if (p.E) {
        E = p.E[c];
    } else {
        E = 0.0;
        for (int s = 0; s < p.n_slots; ++s) E += p.part[(size_t)s * p.nc + c];
    }
    const double T0 = p.T[c];
    double T = T0;
    bool ok = false;
    int it = 0;
    if (E > 0.0 && isfinite(E)) {
        for (it = 1; it <= p.maxit; ++it) {
            const Gsum gs = g_eval(sC, sTh, sW, p.nb, p.W, E, T);
            const double delta = gs.g / gs.gp;
            const double Tn = T - delta;
            if (!(Tn > 0.0) || !isfinite(Tn)) break;
            T = Tn;
            if (fabs(delta) <= p.rtol * T) { ok = true; break; }
        }
        if (!ok) {  // bisection safeguard on a bracket grown from T0
            double lo = T0, hi = T0;
            for (int k = 0; k < 2000 && g_only(sC, sTh, sW, p.nb, p.W, E, lo) > 0.0; ++k) lo *= 0.5;
            for (int k = 0; k < 2000 && g_only(sC, sTh, sW, p.nb, p.W, E, hi) < 0.0; ++k) hi *= 2.0;
            if (g_only(sC, sTh, sW, p.nb, p.W, E, lo) <= 0.0 && g_only(sC, sTh, sW, p.nb, p.W, E, hi) >= 0.0) {
                for (int k = 0; k < 400 && (hi - lo) > p.rtol * hi; ++k) {
                    const double mid = 0.5 * (lo + hi);
                    if (g_only(sC, sTh, sW, p.nb, p.W, E, mid) < 0.0) lo = mid; else hi = mid;
                }
                T = 0.5 * (lo + hi);
                ok = true;
            }
            it = p.maxit + 1;
        }
    }
    if (!ok) {
        atomicExch(p.fail, 1);
        T = T0;
    }
    atomicMax(p.iter_max, it);
    p.T[c] = T;
    const double iT = 1.0 / T;
    for (int k = 0; k < p.nb_loc; ++k) {
        const int b = p.b_lo + k;
        p.i0[(size_t)k * p.nc + c] = sC[b] / expm1(sTh[b] * iT);
    }
}

// E[c] = sum_s part[s][c]  (world > 1: the local partial, all-reduced afterwards)
__global__ void sum_slots_kernel(const double *__restrict__ part, int n_slots, int nc,
                                 double *__restrict__ E) {
    const int c = blockIdx.x * blockDim.x + threadIdx.x;
    if (c >= nc) return;
    double e = 0.0;
    for (int s = 0; s < n_slots; ++s) e += part[(size_t)s * nc + c];
    E[c] = e;
}

// E_loc[c] = sum_{local b} c_b sum_d w_d I[b][d][c] of the current state.
__global__ void energy_kernel(const double *__restrict__ pool, const int32_t *__restrict__ slot,
                              int64_t slab_elems, int nb_loc, int nd, int nc,
                              const double4 *__restrict__ dirs, const double *__restrict__ cw,
                              double *__restrict__ E) {
    const int c = blockIdx.x * blockDim.x + threadIdx.x;
    if (c >= nc) return;
    double e = 0.0;
    for (int k = 0; k < nb_loc; ++k) {
        const double *s = pool + (int64_t)slot[k] * slab_elems;
        double sb = 0.0;
        for (int d = 0; d < nd; ++d) sb = fma(dirs[d].w, s[(size_t)d * nc + c], sb);
        e = fma(cw[k], sb, e);
    }
    E[c] = e;
}

// I0 table of the local rows: i0[k][c] = C_{b_lo+k} / expm1(theta / T_c)
__global__ void i0_table_kernel(const double *__restrict__ T, int nc, int b_lo, int nb_loc,
                                const double *__restrict__ Cb, const double *__restrict__ theta,
                                double *__restrict__ i0) {
    const int c = blockIdx.x * blockDim.x + threadIdx.x;
    if (c >= nc) return;
    const double iT = 1.0 / T[c];
    for (int k = 0; k < nb_loc; ++k)
        i0[(size_t)k * nc + c] = Cb[b_lo + k] / expm1(theta[b_lo + k] * iT);
}

// Equilibrium field I[k][d][c] = i0[k][c] into the current slabs (blockIdx.y = k).
__global__ void equilibrium_kernel(double *__restrict__ pool, const int32_t *__restrict__ slot,
                                   int64_t slab_elems, int nd, int nc,
                                   const double *__restrict__ i0) {
    const int64_t n = (int64_t)nd * nc;
    const int k = blockIdx.y;
    double *s = pool + (int64_t)slot[k] * slab_elems;
    const double *t = i0 + (size_t)k * nc;
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < n;
         e += (int64_t)gridDim.x * blockDim.x)
        s[e] = t[e % nc];
}

// Isothermal ghost table i0w[k][f] = I0_{b_lo+k}(T_wall(f)) (Eq. 6, constant in time).
__global__ void i0w_kernel(const double *__restrict__ twall, int n_iso, int b_lo, int nb_loc,
                           const double *__restrict__ Cb, const double *__restrict__ theta,
                           double *__restrict__ i0w) {
    const int f = blockIdx.x * blockDim.x + threadIdx.x;
    if (f >= n_iso) return;
    for (int k = 0; k < nb_loc; ++k)
        i0w[(size_t)k * n_iso + f] = Cb[b_lo + k] / expm1(theta[b_lo + k] / twall[f]);
}

// S_max = max_{c,d} sum_j max(s_d . g_j(c), 0) (positivity bound of the step).
template <int DIM>
__global__ void outflow_max_kernel(int nc, int mf, int nd, const double *__restrict__ gx,
                                   const double *__restrict__ gy, const double *__restrict__ gz,
                                   const double4 *__restrict__ dirs,
                                   unsigned long long *__restrict__ smax_bits) {
    const int c = blockIdx.x * blockDim.x + threadIdx.x;
    if (c >= nc) return;
    double m = 0.0;
    for (int d = 0; d < nd; ++d) {
        const double4 s = dirs[d];
        double out = 0.0;
        for (int j = 0; j < mf; ++j) {
            const size_t q = (size_t)j * nc + c;
            double a = s.x * gx[q] + s.y * gy[q];
            if (DIM == 3) a += s.z * gz[q];
            out += fmax(a, 0.0);
        }
        m = fmax(m, out);
    }
    atomicMax(smax_bits, (unsigned long long)__double_as_longlong(m));  // m >= 0: bit order = value order
}

// dst[d][u] = src[d][pos[u]]  (internal -> caller cell order), rows of nc.
__global__ void gather_rows_kernel(const double *__restrict__ src, const int32_t *__restrict__ pos,
                                   int nc, int64_t rows, double *__restrict__ dst) {
    const int64_t n = rows * nc;
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < n;
         e += (int64_t)gridDim.x * blockDim.x) {
        const int64_t r = e / nc;
        const int u = (int)(e - r * nc);
        dst[e] = src[r * nc + pos[u]];
    }
}

// dst[d][pos[u]] = src[d][u]  (caller -> internal order)
__global__ void scatter_rows_kernel(const double *__restrict__ src, const int32_t *__restrict__ pos,
                                    int nc, int64_t rows, double *__restrict__ dst) {
    const int64_t n = rows * nc;
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < n;
         e += (int64_t)gridDim.x * blockDim.x) {
        const int64_t r = e / nc;
        const int u = (int)(e - r * nc);
        dst[r * nc + pos[u]] = src[e];
    }
}

}  // namespace bte
