// bte_kernels.cu -- the non-template kernels of the step (temperature solve,
// energy, I0 / rate tables, equilibrium, ghost tables, gathers / scatters,
// halo pack / unpack); declared, with their documentation, in bte_kernels.cuh.
#include "bte_kernels.cuh"

namespace bte {

__global__ void __launch_bounds__(128, 8) newton_kernel(const __grid_constant__ NewtonParams p) {
    if (p.halt && *p.halt) return;
    if (p.done && blockIdx.x == 0 && threadIdx.x == 0) atomicAdd(p.done, 1);
    extern __shared__ double sm[];
    const SolveTables tb = solve_tables(sm, p.nb, p.n_terms);
    load_solve_tables(tb, p);
    __syncthreads();
    const int cl = blockIdx.x * blockDim.x + threadIdx.x;  // chunk-local index
    if (cl >= p.nc) return;
    const int c = p.c_lo + cl;
    double E;
    if (p.E) {
        E = p.E[cl];
    } else {  // the slot sum in sum_slots_kernel's order, bit for bit: partial w sums
              // slots w, w + 8, ... in turn, then the partials in order (8 loads in flight)
        double e[kSumSlotWarps];
#pragma unroll
        for (int w = 0; w < kSumSlotWarps; ++w) e[w] = 0.0;
        for (int s0 = 0; s0 < p.n_slots; s0 += kSumSlotWarps) {
            double v[kSumSlotWarps];
#pragma unroll
            for (int w = 0; w < kSumSlotWarps; ++w)
                v[w] = s0 + w < p.n_slots ? __ldcs(p.part + (size_t)(s0 + w) * p.nc + c) : 0.0;
#pragma unroll
            for (int w = 0; w < kSumSlotWarps; ++w)
                if (s0 + w < p.n_slots) e[w] += v[w];
        }
        E = e[0];
#pragma unroll
        for (int w = 1; w < kSumSlotWarps; ++w) E += e[w];
    }
    const double T0 = p.T[c];
    double Tw = 0.0;
    if (p.td) {
        Tw = p.tr_step ? T0 : p.Tr[c];  // a step: the rate temperature becomes T^n
        if (p.tr_step && !p.tr_now && !p.T_out) p.Tr[c] = T0;  // (chunk solves: newton_finish_kernel stores Tr)
    }
    const Terms t = solve_terms(tb, p, Tw);
    double T = T0;
    bool ok = false, fresh = false;  // fresh: the rows' I0 at the accepted T are stored (or unchanged)
    int it = 0;
    const double *tab = p.i0_t0 ? p.i0_t0 + c : nullptr;  // (I0 at T0 of every row)
    if (E > 0.0 && isfinite(E) && p.single) {  // R3: T + (E - E_eq(T)) / C(T)
        const Gsum gs = tab ? g_eval_table(t, p.W, E, T, tab, p.nc_tab) : g_eval(t, p.W, E, T);
        const double Tn = T - gs.g / gs.gp;
        it = 1;
        if (Tn > 0.0 && isfinite(Tn)) {
            T = Tn;
            ok = true;
        }
    } else if (E > 0.0 && isfinite(E)) {
        // Evaluate g and its derivatives at the iterate (the first from the stored I0
        // table of T^n); accept the iterate once its Newton correction is within
        // rtol T -- its I0 rows were stored by that evaluation (spec) -- else take a
        // Householder step (L555-561: a Newton-type solve of the energy equation)
        for (it = 1; it <= p.maxit; ++it) {
            const bool from_tab = it == 1 && tab, store = p.spec && !from_tab;
            const Gder d = g_eval_der(t, tb, p, E, T, from_tab ? tab : nullptr, p.nc_tab, store, c);
            if (fabs(d.g / d.g1) <= p.racc * T) {
                ok = true;
                fresh = from_tab || store;
                break;
            }
            const double Tn = T - householder_step(d);
            if (!(Tn > 0.0) || !isfinite(Tn)) break;
            T = Tn;
        }
        if (!ok) {  // bisection safeguard on a bracket grown from T0
            double lo = T0, hi = T0;
            for (int k = 0; k < 2000 && g_only(t, p.W, E, lo) > 0.0; ++k) lo *= 0.5;
            for (int k = 0; k < 2000 && g_only(t, p.W, E, hi) < 0.0; ++k) hi *= 2.0;
            if (g_only(t, p.W, E, lo) <= 0.0 && g_only(t, p.W, E, hi) >= 0.0) {
                for (int k = 0; k < 400 && (hi - lo) > p.rtol * hi; ++k) {
                    const double mid = 0.5 * (lo + hi);
                    if (g_only(t, p.W, E, mid) < 0.0) lo = mid; else hi = mid;
                }
                T = 0.5 * (lo + hi);
                ok = true;
            }
            it = p.maxit + 1;
        }
    }
    if (!ok) {
        atomicExch(p.fail, 1);
        T = p.neg_fail ? -T0 : T0;
        fresh = false;
    }
    atomicMax(p.iter_max, it);
    if (p.T_out) {
        p.T_out[c] = T;
        return;
    }
    p.T[c] = T;
    if (p.td && p.tr_now) p.Tr[c] = T;  // (reading 26: the rates follow T)
    const double iT = 1.0 / T;
    for (int k = 0; k < p.nb_loc; ++k) {
        const int b = p.b_lo + k;
        if (!fresh) p.i0[(size_t)k * p.nc + c] = tb.C[b] * (1.0 / expm1(tb.th[b] * iT));  // (= the solve's stores, bitwise)
        if (p.td) p.rate_out[(size_t)k * p.nc + c] = tau_rate(tb.a[b], tb.b[b], tb.r[b], T);
    }
}


__global__ void newton_finish_kernel(const double *__restrict__ Tg, double *__restrict__ T, int nc, int b_lo,
                                     int nb_loc, const double *__restrict__ Cb, const double *__restrict__ theta,
                                     double *__restrict__ i0, int td, const double *__restrict__ ra,
                                     const double *__restrict__ rb, const double *__restrict__ rth,
                                     double *__restrict__ Tr, double *__restrict__ rate_out, int32_t *fail,
                                     const int32_t *__restrict__ halt, int32_t *done, int tr_now,
                                     const int8_t *__restrict__ fresh) {
    if (halt && *halt) return;  // (a solve of an earlier step of the call failed)
    if (done && blockIdx.x == 0 && threadIdx.x == 0) atomicAdd(done, 1);  // the step's last kernel
    const int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (e >= (int64_t)nc * nb_loc) return;
    const int k = (int)(e / nc), c = (int)(e - (int64_t)k * nc);
    double t = Tg[c];
    if (!(t > 0.0)) {
        if (k == 0) atomicExch(fail, 1);
        t = -t;
    }
    if (k == 0) {
        if (td) Tr[c] = tr_now ? t : T[c];  // T^n (lagged rates), or the new T (reading 26)
        T[c] = t;
    }
    const int b = b_lo + k;
    if (!(fresh && fresh[c])) i0[(size_t)k * nc + c] = Cb[b] * (1.0 / expm1(theta[b] * (1.0 / t)));  // (else stored by the solve)
    if (td) rate_out[(size_t)k * nc + c] = tau_rate(ra[b], rb[b], rth[b], t);
}

__global__ void rate_table_kernel(const double *__restrict__ T, int nc, int b_lo, int nb_loc,
                                  const double *__restrict__ ra, const double *__restrict__ rb,
                                  const double *__restrict__ rth, double *__restrict__ out) {
    const int c = blockIdx.x * blockDim.x + threadIdx.x;
    if (c >= nc) return;
    const double t = T[c];
    for (int k = 0; k < nb_loc; ++k) out[(size_t)k * nc + c] = tau_rate(ra[b_lo + k], rb[b_lo + k], rth[b_lo + k], t);
}

// E[c] = sum_s part[s][c]: a block of 8 warps takes 32 cells (lane = cell, so a
// warp's loads are one coalesced 256-byte row of a slot), warp w sums slots
// w, w + 8, ...; the 8 partial sums are added in warp order (deterministic).
__global__ void sum_slots_kernel(const double *__restrict__ part, int n_slots, int nc, double *__restrict__ E,
                                 const int32_t *__restrict__ halt) {
    if (halt && *halt) return;
    __shared__ double red[kSumSlotWarps][32];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int c = blockIdx.x * 32 + lane;
    double e = 0.0;
    if (c < nc) {  // (4 loads in flight per thread, summed in slot order)
        int s = w;
        for (; s + 3 * kSumSlotWarps < n_slots; s += 4 * kSumSlotWarps) {
            double v[4];
#pragma unroll
            for (int u = 0; u < 4; ++u) v[u] = __ldcs(part + (size_t)(s + u * kSumSlotWarps) * nc + c);
#pragma unroll
            for (int u = 0; u < 4; ++u) e += v[u];
        }
        for (; s < n_slots; s += kSumSlotWarps) e += __ldcs(part + (size_t)s * nc + c);
    }
    red[w][lane] = e;
    __syncthreads();
    if (w == 0 && c < nc) {
        double t = red[0][lane];
#pragma unroll
        for (int k = 1; k < kSumSlotWarps; ++k) t += red[k][lane];
        E[c] = t;
    }
}

// E_loc[c] = sum_{local b} c_b sum_d w_d I[b][d][c] of the current state.  A
// block of 8 warps takes 32 cells (lane = cell: each load is a coalesced row of
// a plane); warp w takes directions w, w + 8, ...; the warps' sums are added in
// warp order.  (rate: R2 with the rate law: c_b = rate[k][c] inv_v[k].)
__global__ void energy_kernel(const double *__restrict__ pool, const int32_t *__restrict__ slot,
                              int64_t slab_elems, int ps, int nb_loc, int nd, int nc,
                              const double4 *__restrict__ dirs, const double *__restrict__ cw,
                              const double *__restrict__ rate, const double *__restrict__ inv_v,
                              double *__restrict__ E) {
    __shared__ double red[kSumSlotWarps][32];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int c = blockIdx.x * 32 + lane;
    double e = 0.0;
    if (c < nc)
        for (int k = 0; k < nb_loc; ++k) {
            const double *s = pool + (int64_t)slot[k] * slab_elems + c;
            double sb = 0.0;
            for (int d = w; d < nd; d += kSumSlotWarps) sb = fma(dirs[d].w, s[(size_t)d * ps], sb);
            e = fma(rate ? rate[(size_t)k * nc + c] * inv_v[k] : cw[k], sb, e);
        }
    red[w][lane] = e;
    __syncthreads();
    if (w == 0 && c < nc) {
        double t = red[0][lane];
#pragma unroll
        for (int j = 1; j < kSumSlotWarps; ++j) t += red[j][lane];
        E[c] = t;
    }
}

__global__ void i0_table_kernel(const double *__restrict__ T, int nc, int b_lo, int nb_loc,
                                const double *__restrict__ Cb, const double *__restrict__ theta,
                                double *__restrict__ i0) {
    const int c = blockIdx.x * blockDim.x + threadIdx.x;
    if (c >= nc) return;
    const double iT = 1.0 / T[c];
    for (int k = 0; k < nb_loc; ++k)
        i0[(size_t)k * nc + c] = Cb[b_lo + k] * (1.0 / expm1(theta[b_lo + k] * iT));
}

__global__ void equilibrium_kernel(double *__restrict__ pool, const int32_t *__restrict__ slot,
                                   int64_t slab_elems, int ps, int nd, int nc,
                                   const double *__restrict__ i0) {
    const int64_t n = (int64_t)nd * nc;
    const int k = blockIdx.y;
    double *s = pool + (int64_t)slot[k] * slab_elems;
    const double *t = i0 + (size_t)k * nc;
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < n;
         e += (int64_t)gridDim.x * blockDim.x) {
        const int64_t d = e / nc;
        const int c = (int)(e - d * nc);
        s[d * ps + c] = t[c];
    }
}

__global__ void i0w_kernel(const double *__restrict__ twall, int n_iso, int b_lo, int nb_loc,
                           const double *__restrict__ Cb, const double *__restrict__ theta,
                           double *__restrict__ i0w) {
    const int f = blockIdx.x * blockDim.x + threadIdx.x;
    if (f >= n_iso) return;
    for (int k = 0; k < nb_loc; ++k)
        i0w[(size_t)k * n_iso + f] = Cb[b_lo + k] / expm1(theta[b_lo + k] / twall[f]);
}

__global__ void side_table_kernel(const double *__restrict__ i0w, int n_iso, const int32_t *__restrict__ col,
                                  int n_side, int nb_loc, double *__restrict__ out) {
    const int64_t n = (int64_t)n_side * nb_loc;
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < n; e += (int64_t)gridDim.x * blockDim.x) {
        const int64_t k = e / n_side;
        const int c = col[e - k * n_side];
        out[e] = c >= 0 ? i0w[k * n_iso + c] : 0.0;
    }
}

__global__ void gather_rows_kernel(const double *__restrict__ src, const int32_t *__restrict__ pos,
                                   int nc, int64_t stride, int64_t rows, double *__restrict__ dst) {
    const int64_t n = rows * nc;
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < n;
         e += (int64_t)gridDim.x * blockDim.x) {
        const int64_t r = e / nc;
        const int u = (int)(e - r * nc);
        dst[e] = src[r * stride + pos[u]];
    }
}

__global__ void scatter_rows_kernel(const double *__restrict__ src, const int32_t *__restrict__ pos,
                                    int nc, int64_t stride, int64_t rows, double *__restrict__ dst) {
    const int64_t n = rows * nc;
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < n;
         e += (int64_t)gridDim.x * blockDim.x) {
        const int64_t r = e / nc;
        const int u = (int)(e - r * nc);
        dst[r * stride + pos[u]] = src[e];
    }
}

__global__ void halo_pack_kernel(const __grid_constant__ HaloParams p, double *__restrict__ buf) {
    if (p.fail && *p.fail) return;
    const int64_t per = (int64_t)p.n_dirs * p.n;
    const int k = blockIdx.y;
    const double *s = p.row[k];
    double *o = buf + k * per;
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < per; e += (int64_t)gridDim.x * blockDim.x) {
        const int j = (int)(e / p.n);
        const int i = (int)(e - (int64_t)j * p.n);
        o[e] = s[(int64_t)__ldg(p.dirs + j) * p.ps + __ldg(p.cells + i)];
    }
}

__global__ void halo_unpack_kernel(const __grid_constant__ HaloParams p, const double *__restrict__ buf) {
    if (p.fail && *p.fail) return;
    const int64_t per = (int64_t)p.n_dirs * p.n;
    const int k = blockIdx.y;
    double *s = p.row[k];
    const double *in = buf + k * per;
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < per; e += (int64_t)gridDim.x * blockDim.x) {
        const int j = (int)(e / p.n);
        const int i = (int)(e - (int64_t)j * p.n);
        s[(int64_t)__ldg(p.dirs + j) * p.ps + __ldg(p.cells + i)] = in[e];
    }
}

}  // namespace bte
