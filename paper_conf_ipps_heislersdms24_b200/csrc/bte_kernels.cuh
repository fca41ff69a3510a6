// bte_kernels.cuh -- sm_100a kernels of the explicit phonon-BTE step
// (templates, device helpers, parameter blocks; the non-template kernels are
// defined in bte_kernels.cu).
//
// Paper: E. Heisler et al., IPDPS 2024; "Lnnn" = line of PAPER.md.
//
// Every flux kernel computes the Eq. 3 / Eq. 5 forward-Euler update with the
// first-order upwind face flux (L264-292, L529-553, L644-647), the RTA source
// (I0 - I)/tau, the Eq. 6 ghosts on boundary faces (L563-607) and the fused
// per-cell energy partial sum_b c_b sum_d w_d I' (L412-418).  HBM-bound: 16 B
// per (cell, dir, band) update (read I^n, write I^{n+1}).
//   flux_box_kernel          structured 2-D / 3-D grids (the paper's meshes):
//                            z-marching 32 x 8 tiles, tensor-copied halo boxes
//   flux_tma_kernel          any mesh whose faces come in opposite pairs: 256-cell
//                            tiles staged by bulk copies
//   flux_tma_generic_kernel  any face-based mesh (triangles, split faces): tile +
//                            halo + ghosts staged by the producer warp
//   flux_kernel              register-pipelined fallback (generic faces)
//   newton_kernel / newton_lanes_kernel / newton_finish_kernel
//                            per-cell temperature from the energy (L407-418,
//                            L555-561, L707-716) and the I0 table of the next step
//   small kernels            slot sums, reductions, gathers / scatters into caller
//                            cell order, equilibrium initialisation, ghost tables,
//                            dt bound, halo pack / unpack
//
// Layout: the slab of band-row b = [n_dirs][plane stride] doubles
// in a slab pool (cell fastest); per-cell face geometry in struct-of-arrays
// face slots [j][cell]: nbr (int32), g = (A_f / V_c) n_f (FP64), face codes.
#pragma once
#include <cstdint>
#include <cuda.h>  // CUtensorMap (box kernel tensor maps)
#include <cuda_runtime.h>

namespace bte {

constexpr int kMaxBandsPerLaunch = 128;  // band-rows per rank
constexpr int kMaxBands = 1024;          // band-rows in all (the warp temperature solve: 32 per lane)
constexpr int kMaxThreads = 256;
#ifndef BTE_MIN_BLOCKS
#define BTE_MIN_BLOCKS 2  // resident 256-thread blocks per SM the flux kernels are compiled for
#endif

enum : int8_t { kFaceInterior = 0, kFaceIso = 1, kFaceSym = 2 };

struct FluxParams {
    int32_t nc;          // cells
    int32_t ps;          // plane stride (nc padded to 32)
    int32_t nd;          // directions
    int32_t dchunk;      // directions per block
    int32_t n_dchunks;
    int32_t nbl;         // band-rows in this launch (a multiple of the template BG)
    int32_t band0;       // rank-local index of the launch's first band-row
    int32_t slot0;       // first energy-partial slot of this launch
    const double *i0;    // [nb_loc][nc]  I0_b(T_c) of the current step
    double *part;        // [n_slots][nc] energy partials
    // Face slots, struct-of-arrays [slot][nc].  Generic: one slot per face.
    // Paired: one slot per opposite face pair; nbr describes the "+" face (the
    // one whose g is stored), nbm the "-" face (g_- = -g_+).  For a boundary
    // face nbr holds its isothermal-table column (isothermal) or is unused
    // (specular); the face kind is in fcode.
    const int32_t *nbr, *nbm;
    const double *gx, *gy, *gz;  // g = (A_f / V_c) n_f
    double gu[3][3];             // uniform-geometry meshes: g of pair q (same for every cell)
    const uint32_t *fcode;       // paired [nc]: 5-bit code per side (pair q: bits 10q "+", 10q+5 "-")
    const uint8_t *fcode8;       // generic [MF][nc]: code per face
    const int32_t *refl;         // [n_classes][nd] reflected direction of a specular class
    const double *i0w;           // [nb_loc][n_iso]  I0_b(T_wall) per isothermal face
    int32_t n_iso;
    const double4 *dirs;         // [nd] {s_x, s_y, s_z, w}
    double dt;
    // temperature-dependent relaxation times (N1, generic kernel only):
    // rate_cur / rate_next [nb_loc][nc] = 1/tau at the rate temperature of this
    // step / at T^n (the R2 energy weight rate_next / v_b); nullptr: constants
    const double *rate_cur, *rate_next;
    int32_t rate_r2;                           // R2 weights from rate_next (else cw)
    double inv_v[kMaxBandsPerLaunch];          // 1 / v_b
    const double *in_ptr[kMaxBandsPerLaunch];  // per launch-local band-row: input slab (I^n)
    double *out_ptr[kMaxBandsPerLaunch];       // ... output slab (I^{n+1})
    double dtit[kMaxBandsPerLaunch];           // dt / tau_b
    double kv[kMaxBandsPerLaunch];             // dt v_b
    double cw[kMaxBandsPerLaunch];             // temperature weight c_b
    // TMA-staged generic-face kernel: per tile (256 cells) the out-of-tile
    // upwind cells its interior faces read and its boundary faces' ghosts,
    // gathered into the stage behind the tile's own values (at host-chosen
    // positions >= kTile); per face slot the shared-memory index of its upwind value
    const int32_t *hl_off;   // [n_tiles + 1] halo cells of tile t: [hl_off[t], hl_off[t+1])
    const int32_t *hl_cell;  // plane columns of the halo cells
    const int32_t *hl_pos;   // their staged positions
    const int32_t *bl_off;   // [n_tiles + 1] boundary-face ghosts of tile t
    const int32_t *bl_col;   // specular: the cell's column; isothermal: the I0w table column
    const int32_t *bl_cls;   // specular class (reflected direction refl[cls][d]); -1: isothermal
    const int32_t *bl_pos;   // their staged positions
    const uint16_t *sidx;    // [MF][nc] staged index: own tile < kTile <= halo and ghosts
    int32_t hstride;         // doubles per staged band-row: kTile + halo + ghost capacity
    // ENOCONV stop (bte_step): fail != 0 once a temperature solve of an earlier
    // step of the call failed; the flux launch is then a no-op and block 0
    // latches the flag into halt, which the rest of the step's kernels read
    const int32_t *fail;
    int32_t *halt;
};

// The stop guard at the top of every flux launch (uniform per launch).
__device__ __forceinline__ bool flux_halted(const int32_t *fail, int32_t *halt) {
    const int f = fail ? *fail : 0;
    if (halt && blockIdx.x == 0 && blockIdx.y == 0 && threadIdx.x == 0) *halt = f;
    return f != 0;
}

__device__ __forceinline__ double4 load_dir(const double4 *dirs, int d) {
    const double2 a = __ldg(reinterpret_cast<const double2 *>(dirs + d));
    const double2 b = __ldg(reinterpret_cast<const double2 *>(dirs + d) + 1);
    return make_double4(a.x, a.y, b.x, b.y);
}

// Face codes (Eq. 6: the upwind value entering through a face):
//   kCodeInterior  I^n[b][d][nbr]            (same plane)
//   kCodeIso       I0_b(T_wall) = I0w[b][nbr] (isothermal table column)
//   0..15          specular class k: I^n[b][r_k(d)][c] (reflected direction,
//                  same cell, old level) = same plane + (r_k(d) - d) * ps + c - c
// Paired layout: 5-bit codes; generic layout: 8-bit codes.
constexpr uint32_t kCodeInterior = 31;
constexpr uint32_t kCodeIso = 16;
constexpr int kMaxPairedClasses = 16;
constexpr uint32_t kCode8Interior = 255;
constexpr uint32_t kCode8Iso = 254;
constexpr int kMaxGenericClasses = 254;

// ---------------------------------------------------------------------------
// One thread owns one cell and a (band group, direction chunk) of its
// unknowns.  Per direction it forms alpha_j = s_d . g_j (g_j = A_j/V n_j) once
// for the BG band-rows, issues every load of the iteration (own value and the
// inflow faces' upwind values of all BG rows) before using any, then writes
//   I' = I (1 - dt/tau - dt v out) + (dt/tau) I0 - dt v sum_{alpha<0} alpha I_up
// (Eq. 3/5, L269-292, L546-553; upwind L264-267) with a streaming store and
// accumulates c_b w_d I' for the energy partial (L412-418).  Cells with a
// boundary face (has_bnd) take the face-kind path; for the others it is a
// warp-uniform skip.
//
// Generic connectivity: up to MF faces per cell, each with its own neighbour.
template <int DIM, int MF, int BG>
__global__ void __launch_bounds__(kMaxThreads, BTE_MIN_BLOCKS)
flux_kernel(const __grid_constant__ FluxParams p) {
    if (flux_halted(p.fail, p.halt)) return;
    const int c = blockIdx.x * blockDim.x + threadIdx.x;
    if (c >= p.nc) return;
    const int grp = blockIdx.y / p.n_dchunks;
    const int dch = blockIdx.y - grp * p.n_dchunks;
    const int lg0 = grp * BG;  // launch-local first band-row of the group (groups are full)
    const int d0 = dch * p.dchunk;
    const int d1 = min(p.nd, d0 + p.dchunk);
    const int nc = p.nc;
    const int ps = p.ps;

    int nbr[MF];
    uint32_t code[MF];
    double gx[MF], gy[MF], gz[MF];
    bool has_bnd = false;
#pragma unroll
    for (int j = 0; j < MF; ++j) {
        const int q = j * nc + c;
        nbr[j] = __ldg(p.nbr + q);
        gx[j] = __ldg(p.gx + q);
        gy[j] = __ldg(p.gy + q);
        gz[j] = DIM == 3 ? __ldg(p.gz + q) : 0.0;
        code[j] = __ldg(p.fcode8 + q);
        has_bnd |= code[j] != kCode8Interior;
    }
    double src[BG], dtk[BG], cwk[BG];
#pragma unroll
    for (int k = 0; k < BG; ++k) {  // dt/tau I0_b(T_c); the cell's rates with the rate law
        const int64_t row = (int64_t)(p.band0 + lg0 + k) * nc + c;
        dtk[k] = p.rate_cur ? p.dt * __ldg(p.rate_cur + row) : p.dtit[lg0 + k];
        cwk[k] = (p.rate_cur && p.rate_r2) ? __ldg(p.rate_next + row) * p.inv_v[lg0 + k] : p.cw[lg0 + k];
        src[k] = dtk[k] * __ldg(p.i0 + row);
    }
    double e = 0.0;
    for (int d = d0; d < d1; ++d) {
        const double4 sd = load_dir(p.dirs, d);
        double a[MF];
        int idx[MF];
        double out = 0.0;
#pragma unroll
        for (int j = 0; j < MF; ++j) {
            a[j] = DIM == 3 ? fma(sd.z, gz[j], fma(sd.y, gy[j], sd.x * gx[j])) : fma(sd.y, gy[j], sd.x * gx[j]);
            out += fmax(a[j], 0.0);  // outflow faces carry the cell's own value
            idx[j] = nbr[j];
        }
        if (has_bnd) {
#pragma unroll
            for (int j = 0; j < MF; ++j)
                if (code[j] < kCode8Iso) idx[j] = (__ldg(p.refl + code[j] * p.nd + d) - d) * ps + c;
        }
        const int64_t po = (int64_t)d * ps;
        double ic[BG], nv[BG][MF];
#pragma unroll
        for (int k = 0; k < BG; ++k) {  // every load of the iteration first
            const double *pl = p.in_ptr[lg0 + k] + po;
            ic[k] = __ldg(pl + c);
            if (!has_bnd) {
#pragma unroll
                for (int j = 0; j < MF; ++j) nv[k][j] = a[j] < 0.0 ? __ldg(pl + idx[j]) : 0.0;
            } else {
                const double *iso = p.i0w + (int64_t)(p.band0 + lg0 + k) * p.n_iso;
#pragma unroll
                for (int j = 0; j < MF; ++j)
                    nv[k][j] = a[j] < 0.0 ? __ldg((code[j] == kCode8Iso ? iso : pl) + idx[j]) : 0.0;
            }
        }
#pragma unroll
        for (int k = 0; k < BG; ++k) {
            double infl = 0.0;
#pragma unroll
            for (int j = 0; j < MF; ++j) infl = fma(fmin(a[j], 0.0), nv[k][j], infl);
            const double kv = p.kv[lg0 + k];
            const double inew = fma(ic[k], (1.0 - dtk[k]) - kv * out, fma(-kv, infl, src[k]));
            __stcs(p.out_ptr[lg0 + k] + po + c, inew);
            e = fma(cwk[k] * sd.w, inew, e);
        }
    }
    p.part[(int64_t)(p.slot0 + grp * p.n_dchunks + dch) * nc + c] = e;
}

// ---------------------------------------------------------------------------
// TMA-staged paired kernel (sm_100a bulk-copy engine + mbarriers).
//
// A block is one tile of kTile = 256 consecutive cells (with the Morton hint:
// an 8x8x4 brick).  For every (band-row, direction) plane the tile's own
// values are one contiguous 2 KB segment, so one elected thread streams them
// into a kStages-deep shared-memory ring with cp.async.bulk (completion counted
// on an mbarrier), kStages iterations ahead of the compute.  Upwind neighbours
// inside the tile are read from the staged segment; only halo neighbours,
// specular faces (another direction's plane) and isothermal faces (the I0w
// table) are global loads, issued at the top of the iteration.  Arithmetic is
// the same as flux_kernel's with opposite-face pairs (one inflow face per pair).
constexpr int kTile = 256;
#ifndef BTE_TMA_STAGES
#define BTE_TMA_STAGES 4
#endif
constexpr int kStages = BTE_TMA_STAGES;  // shared-memory ring depth (iterations in flight)

__device__ __forceinline__ uint32_t smem_u32(const void *ptr) {
    return (uint32_t)__cvta_generic_to_shared(ptr);
}
__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t *bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ bool mbar_try_wait(uint64_t *bar, uint32_t phase) {
    uint32_t ok;
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(ok)
        : "r"(smem_u32(bar)), "r"(phase)
        : "memory");
    return ok != 0;
}
__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, uint32_t bytes, uint64_t *bar) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
            smem_u32(dst)),
        "l"(src), "r"(bytes), "r"(smem_u32(bar))
        : "memory");
}

// Warp-specialised: warps 0..7 compute (one cell each), warp 8 is the producer.
// full[s] completes when stage s has landed (tx bytes); empty[s] completes when
// all 8 compute warps are done with it -- no block-wide barrier in the loop.
constexpr int kComputeWarps = kTile / 32;
constexpr int kTmaThreads = kTile + 32;

__device__ __forceinline__ void mbar_arrive(uint64_t *bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}

// Shared-memory direction table of a block's chunk (uniform geometry): per
// direction out = sum |s.g_q|, -|s.g_q| per pair, w_d, and the upwind side bits.
template <int NP>
struct DirEntry {
    double out, amin[NP], w;
    uint32_t up;  // bit q: s.g_q > 0 (inflow through the "-" face)
};

template <int DIM, int NP>
__device__ __forceinline__ DirEntry<NP> dir_entry(const FluxParams &p, int d) {
    const double4 sd = load_dir(p.dirs, d);
    DirEntry<NP> t;
    t.out = 0.0;
    t.up = 0;
#pragma unroll
    for (int q = 0; q < NP; ++q) {
        const double a = DIM == 3 ? fma(sd.z, p.gu[q][2], fma(sd.y, p.gu[q][1], sd.x * p.gu[q][0]))
                                  : fma(sd.y, p.gu[q][1], sd.x * p.gu[q][0]);
        t.out += fabs(a);
        t.amin[q] = -fabs(a);
        t.up |= (a > 0.0 ? 1u : 0u) << q;
    }
    t.w = sd.w;
    return t;
}

template <int DIM, int NP, int BG, bool UG>
__global__ void __launch_bounds__(kTmaThreads, BTE_MIN_BLOCKS)
flux_tma_kernel(const __grid_constant__ FluxParams p) {
    extern __shared__ __align__(128) double ring[];  // [kStages][BG][kTile], then (UG) DirEntry[dchunk]
    __shared__ __align__(8) uint64_t full[kStages];
    __shared__ __align__(8) uint64_t empty[kStages];
    if (flux_halted(p.fail, p.halt)) return;
    const int tid = threadIdx.x;
    const int tile0 = blockIdx.x * kTile;
    const int grp = blockIdx.y / p.n_dchunks;
    const int dch = blockIdx.y - grp * p.n_dchunks;
    const int lg0 = grp * BG;
    const int d0 = dch * p.dchunk;
    const int nit = min(p.nd, d0 + p.dchunk) - d0;
    const int nc = p.nc;
    const int ps = p.ps;
    constexpr uint32_t kBytes = BG * kTile * sizeof(double);

    DirEntry<NP> *dtab = reinterpret_cast<DirEntry<NP> *>(ring + kStages * BG * kTile);
    if (tid == 0) {
#pragma unroll
        for (int s = 0; s < kStages; ++s) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], kComputeWarps);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (UG)
        for (int i = tid; i < nit; i += kTmaThreads) dtab[i] = dir_entry<DIM, NP>(p, d0 + i);
    __syncthreads();

    if (tid >= kTile) {  // ------------------------------------------ producer warp
        if (tid == kTile) {
            for (int i = 0; i < nit; ++i) {
                const int st = i % kStages;
                if (i >= kStages)
                    while (!mbar_try_wait(&empty[st], ((i / kStages) - 1) & 1)) {
                    }
                mbar_arrive_expect_tx(&full[st], kBytes);
                const int64_t off = (int64_t)(d0 + i) * ps + tile0;
#pragma unroll
                for (int k = 0; k < BG; ++k)
                    bulk_g2s(ring + (st * BG + k) * kTile, p.in_ptr[lg0 + k] + off, kTile * sizeof(double), &full[st]);
            }
        }
        return;
    }

    // --------------------------------------------------------------- compute warps
    const int c = tile0 + tid;
    const bool valid = c < nc;
    const int lane = tid & 31;
    int np_[NP], nm_[NP];
    double gx[NP], gy[NP], gz[NP];
    uint32_t codes = (1u << (10 * NP)) - 1u;
    double src[BG];
#pragma unroll
    for (int q = 0; q < NP; ++q) {
        const int o = q * nc + c;
        np_[q] = valid ? __ldg(p.nbr + o) : c;
        nm_[q] = valid ? __ldg(p.nbm + o) : c;
        if (!UG) {
            gx[q] = valid ? __ldg(p.gx + o) : 0.0;
            gy[q] = valid ? __ldg(p.gy + o) : 0.0;
            gz[q] = (DIM == 3 && valid) ? __ldg(p.gz + o) : 0.0;
        }
    }
    if (valid) codes = __ldg(p.fcode + c);
    const bool has_bnd = codes != (1u << (10 * NP)) - 1u;
#pragma unroll
    for (int k = 0; k < BG; ++k)
        src[k] = valid ? p.dtit[lg0 + k] * __ldg(p.i0 + (int64_t)(p.band0 + lg0 + k) * nc + c) : 0.0;

    double e = 0.0;
    for (int i = 0; i < nit; ++i) {
        const int d = d0 + i;
        double amin[NP], out, wd;
        uint32_t up = 0;
        if (UG) {  // block-uniform: from the shared-memory direction table
            const DirEntry<NP> &t = dtab[i];
            out = t.out;
            wd = t.w;
            up = t.up;
#pragma unroll
            for (int q = 0; q < NP; ++q) amin[q] = t.amin[q];
        } else {
            const double4 sd = load_dir(p.dirs, d);
            out = 0.0;
            wd = sd.w;
#pragma unroll
            for (int q = 0; q < NP; ++q) {
                const double a = DIM == 3 ? fma(sd.z, gz[q], fma(sd.y, gy[q], sd.x * gx[q])) : fma(sd.y, gy[q], sd.x * gx[q]);
                out += fabs(a);
                amin[q] = -fabs(a);
                up |= (a > 0.0 ? 1u : 0u) << q;
            }
        }
        int idx[NP];
        bool glob[NP], iso[NP];
#pragma unroll
        for (int q = 0; q < NP; ++q) {
            const bool plus_out = (up >> q) & 1u;
            idx[q] = plus_out ? nm_[q] : np_[q];
            iso[q] = false;
            if (has_bnd) {
                const uint32_t cd = (codes >> (10 * q + (plus_out ? 5 : 0))) & kCodeInterior;
                iso[q] = cd == kCodeIso;
                if (cd < kCodeIso) idx[q] = (__ldg(p.refl + cd * p.nd + d) - d) * ps + c;
            }
            glob[q] = iso[q] || (unsigned)(idx[q] - tile0) >= (unsigned)kTile;
        }
        // halo / boundary values: global loads first (overlap the stage wait)
        const int64_t po = (int64_t)d * ps;
        double nv[BG][NP];
#pragma unroll
        for (int k = 0; k < BG; ++k) {
            const double *pl = p.in_ptr[lg0 + k] + po;
            const double *isot = p.i0w + (int64_t)(p.band0 + lg0 + k) * p.n_iso;
#pragma unroll
            for (int q = 0; q < NP; ++q)
                nv[k][q] = (valid && glob[q]) ? __ldg((iso[q] ? isot : pl) + idx[q]) : 0.0;
        }
        const int st = i % kStages;
        while (!mbar_try_wait(&full[st], (i / kStages) & 1)) {
        }
        const double *stage = ring + st * BG * kTile;
        double inew[BG];
#pragma unroll
        for (int k = 0; k < BG; ++k) {
            const double *sk = stage + k * kTile;
            const double ic = sk[tid];
            double infl = 0.0;
#pragma unroll
            for (int q = 0; q < NP; ++q) infl = fma(amin[q], glob[q] ? nv[k][q] : sk[idx[q] - tile0], infl);
            const double kv = p.kv[lg0 + k];
            inew[k] = fma(ic, (1.0 - p.dtit[lg0 + k]) - kv * out, fma(-kv, infl, src[k]));
        }
        __syncwarp();
        if (lane == 0) mbar_arrive(&empty[st]);  // this warp is done with the stage
#pragma unroll
        for (int k = 0; k < BG; ++k) {
            if (valid) __stcs(p.out_ptr[lg0 + k] + po + c, inew[k]);
            e = fma(p.cw[lg0 + k] * wd, inew[k], e);
        }
    }
    if (valid) p.part[(int64_t)(p.slot0 + grp * p.n_dchunks + dch) * nc + c] = e;
}

// ---------------------------------------------------------------------------
// TMA-staged kernel for general meshes (unstructured: triangles, split faces,
// any face-based mesh).  One 256-cell tile of the locality
// order per block.  For every (band-row, direction) plane the producer warp
// stages, kStagesG iterations ahead, everything the tile's faces read: the
// tile's own 2 KB segment (lane 0, cp.async.bulk), its halo -- the out-of-tile
// cells its interior faces point to -- and the Eq. 6 ghosts of its boundary
// faces (isothermal: I0_b(T_wall) from the table; specular: the same cell's
// value in the reflected direction's plane), both gathered by the 32 lanes with
// 8-byte cp.async whose completion the same mbarrier tracks
// (cp.async.mbarrier.arrive.noinc).  The lists are built on the host.  The
// compute warps then read every upwind value from shared memory at a
// host-computed index: no global loads and no boundary branch in the update.
// Arithmetic of flux_kernel: up to MF faces per cell, outflow
// sum_j max(alpha_j, 0), inflow sum_j min(alpha_j, 0) I_up (Eq. 3/5), with the
// rate law the cell's own rates.
#ifndef BTE_TMA_GENERIC_STAGES
#define BTE_TMA_GENERIC_STAGES 3  // measured on B200 (C3t): 3 > 6 > 12 stages
#endif
constexpr int kStagesG = BTE_TMA_GENERIC_STAGES;
constexpr int kMaxTileStaged = 768;  // halo + ghost values per tile (else the register kernel)

__device__ __forceinline__ void cp_async_8(void *dst, const void *src) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async_mbar_arrive(uint64_t *bar) {
    asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];" ::"r"(smem_u32(bar)) : "memory");
}

#ifndef BTE_TMA_GENERIC_MIN_BLOCKS
#define BTE_TMA_GENERIC_MIN_BLOCKS 3
#endif
// HS: the staged band-row stride in doubles when fixed at compile time (the
// common case kTileStagedFixed: the row offsets become load immediates), 0: p.hstride.
constexpr int kTileStagedFixed = kTile + 128;
template <int DIM, int MF, int BG, bool TD, int HS>
__global__ void __launch_bounds__(kTmaThreads, BTE_TMA_GENERIC_MIN_BLOCKS)
flux_tma_generic_kernel(const __grid_constant__ FluxParams p) {
    // [kStagesG][BG][hstride] ring, double4 dirs[dchunk], then the tile's staging
    // lists: halo columns and positions [nh], ghost columns, classes, positions [ng]
    extern __shared__ __align__(128) double ring[];
    __shared__ __align__(8) uint64_t full[kStagesG];
    __shared__ __align__(8) uint64_t empty[kStagesG];
    if (flux_halted(p.fail, p.halt)) return;
    const int tid = threadIdx.x;
    const int tile0 = blockIdx.x * kTile;
    const int grp = blockIdx.y / p.n_dchunks;
    const int dch = blockIdx.y - grp * p.n_dchunks;
    const int lg0 = grp * BG;
    const int nrows = min(BG, p.nbl - lg0);  // (a ragged last group: rows k >= nrows idle)
    const int d0 = dch * p.dchunk;
    const int nit = min(p.nd, d0 + p.dchunk) - d0;
    const int nc = p.nc;
    const int ps = p.ps;
    const int hs = HS ? HS : p.hstride;
    double4 *sdir = reinterpret_cast<double4 *>(ring + kStagesG * BG * hs);  // this chunk's {s, w}
    int32_t *shl = reinterpret_cast<int32_t *>(sdir + p.dchunk);          // halo columns
    const int h0 = __ldg(p.hl_off + blockIdx.x), nh = __ldg(p.hl_off + blockIdx.x + 1) - h0;
    const int g0 = __ldg(p.bl_off + blockIdx.x), ng = __ldg(p.bl_off + blockIdx.x + 1) - g0;
    int32_t *shp = shl + nh, *sgc = shp + nh, *sgk = sgc + ng, *sgp = sgk + ng;

    if (tid == 0) {
#pragma unroll
        for (int s = 0; s < kStagesG; ++s) {
            mbar_init(&full[s], 1 + 32);  // lane 0's expect-tx arrive + one async arrive per producer lane
            mbar_init(&empty[s], kComputeWarps);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    for (int i = tid; i < nit; i += kTmaThreads) sdir[i] = load_dir(p.dirs, d0 + i);
    // the tile's lists, read once per block (every plane of the block gathers the same cells)
    for (int i = tid; i < nh; i += kTmaThreads) {
        shl[i] = __ldg(p.hl_cell + h0 + i);
        shp[i] = __ldg(p.hl_pos + h0 + i);
    }
    for (int i = tid; i < ng; i += kTmaThreads) {
        sgc[i] = __ldg(p.bl_col + g0 + i);
        sgk[i] = __ldg(p.bl_cls + g0 + i);
        sgp[i] = __ldg(p.bl_pos + g0 + i);
    }
    __syncthreads();

    if (tid >= kTile) {  // ------------------------------------------ producer warp
        const int lane = tid - kTile;
        int st = 0;
        uint32_t ph = 0;
        for (int i = 0; i < nit; ++i) {
            const int d = d0 + i;
            if (i >= kStagesG)
                while (!mbar_try_wait(&empty[st], ph ^ 1u)) {
                }
            const int64_t po = (int64_t)d * ps;
            double *sbase = ring + st * BG * hs;
            if (lane == 0) {
                mbar_arrive_expect_tx(&full[st], (uint32_t)(nrows * kTile * sizeof(double)));
#pragma unroll
                for (int k = 0; k < BG; ++k)
                    if (k < nrows)
                        bulk_g2s(sbase + k * hs, p.in_ptr[lg0 + k] + po + tile0, kTile * sizeof(double), &full[st]);
            }
            for (int h = lane; h < nh; h += 32) {  // halo: neighbour cells outside the tile
                const int col = shl[h], pos = shp[h];
#pragma unroll
                for (int k = 0; k < BG; ++k)
                    if (k < nrows) cp_async_8(sbase + k * hs + pos, p.in_ptr[lg0 + k] + po + col);
            }
            for (int g = lane; g < ng; g += 32) {  // boundary-face ghosts (Eq. 6, old level)
                const int col = sgc[g], cls = sgk[g], pos = sgp[g];
                const int64_t off = cls < 0 ? (int64_t)col
                                            : (int64_t)__ldg(p.refl + cls * p.nd + d) * ps + col;
#pragma unroll
                for (int k = 0; k < BG; ++k)
                    if (k < nrows)
                    cp_async_8(sbase + k * hs + pos,
                               (cls < 0 ? p.i0w + (int64_t)(p.band0 + lg0 + k) * p.n_iso : p.in_ptr[lg0 + k]) + off);
            }
            cp_async_mbar_arrive(&full[st]);
            if (++st == kStagesG) st = 0, ph ^= 1u;
        }
        return;
    }

    // --------------------------------------------------------------- compute warps
    const int c = tile0 + tid;
    const bool valid = c < nc;
    const int lane = tid & 31;
    uint32_t sxb[MF];  // byte offset (in a staged band-row) of each face's upwind value
    double gx[MF], gy[MF], gz[MF];
#pragma unroll
    for (int j = 0; j < MF; ++j) {
        const int q = j * nc + c;
        sxb[j] = 8u * (valid ? (uint32_t)__ldg(p.sidx + q) : (uint32_t)tid);
        gx[j] = valid ? __ldg(p.gx + q) : 0.0;
        gy[j] = valid ? __ldg(p.gy + q) : 0.0;
        gz[j] = (DIM == 3 && valid) ? __ldg(p.gz + q) : 0.0;
    }
    uint32_t ownb = 8u * (uint32_t)tid;
#pragma unroll
    for (int j = 0; j < MF; ++j) asm volatile("" : "+r"(sxb[j]));  // (loads address [offset + row base])
    asm volatile("" : "+r"(ownb));
    const uint32_t rowb = 8u * (uint32_t)hs;  // bytes per staged band-row (HS: a constant)
    // dt/tau I0_b(T_c); TD (rate law): the cell's own rates, else the band's constants
    double src[BG], dtk[TD ? BG : 1], cwk[TD ? BG : 1];
#pragma unroll
    for (int k = 0; k < BG; ++k) {
        const int64_t row = (int64_t)(p.band0 + lg0 + min(k, nrows - 1)) * nc + c;  // (idle rows: a valid row)
        if (TD) {
            dtk[k] = valid ? p.dt * __ldg(p.rate_cur + row) : 0.0;
            cwk[k] = (p.rate_r2 && valid) ? __ldg(p.rate_next + row) * p.inv_v[lg0 + k] : p.cw[lg0 + k];
        }
        src[k] = valid ? (TD ? dtk[k] : p.dtit[lg0 + k]) * __ldg(p.i0 + row) : 0.0;
    }
    double *op[BG];  // this cell's output in the chunk's first plane, one plane per iteration on
#pragma unroll
    for (int k = 0; k < BG; ++k) op[k] = p.out_ptr[lg0 + min(k, nrows - 1)] + (int64_t)d0 * ps + c;

    double e = 0.0;
    int st = 0;
    uint32_t ph = 0;
    for (int i = 0; i < nit; ++i) {
        const double4 sd = sdir[i];
        double am[MF];  // min(alpha_j, 0): the inflow weights
        double out = 0.0;
#pragma unroll
        for (int j = 0; j < MF; ++j) {
            const double a = DIM == 3 ? fma(sd.z, gz[j], fma(sd.y, gy[j], sd.x * gx[j])) : fma(sd.y, gy[j], sd.x * gx[j]);
            am[j] = a > 0.0 ? 0.0 : a;  // (select)
            out += a - am[j];           // max(alpha_j, 0), exactly: outflow faces carry the cell's own value
        }
        while (!mbar_try_wait(&full[st], ph)) {
        }
        const char *const cb = reinterpret_cast<const char *>(ring + st * BG * hs);
        // per face one address (stage + offset); the band-rows are k row strides on
        const char *fa[MF];
#pragma unroll
        for (int j = 0; j < MF; ++j) fa[j] = cb + sxb[j];
        const char *const oa = cb + ownb;
        auto at = [](const char *a, uint32_t b) { return *reinterpret_cast<const double *>(a + b); };
        double inew[BG];
#pragma unroll
        for (int k = 0; k < BG; ++k) {
            if (k >= nrows) { inew[k] = 0.0; continue; }  // (idle row of a ragged group)
            double infl = 0.0;
#pragma unroll
            for (int j = 0; j < MF; ++j) infl = fma(am[j], at(fa[j], k * rowb), infl);
            const double kv = p.kv[lg0 + k];
            const double dt_tau = TD ? dtk[k] : p.dtit[lg0 + k];
            inew[k] = fma(at(oa, k * rowb), (1.0 - dt_tau) - kv * out, fma(-kv, infl, src[k]));
        }
        __syncwarp();
        if (lane == 0) mbar_arrive(&empty[st]);  // this warp is done with the stage
        if (++st == kStagesG) st = 0, ph ^= 1u;
#pragma unroll
        for (int k = 0; k < BG; ++k) {
            if (k >= nrows) continue;
            if (valid) __stcs(op[k], inew[k]);
            op[k] += ps;
            e = fma((TD ? cwk[k] : p.cw[lg0 + k]) * sd.w, inew[k], e);
        }
    }
    if (valid) p.part[(int64_t)(p.slot0 + grp * p.n_dchunks + dch) * nc + c] = e;
}

// ---------------------------------------------------------------------------
// Box kernel: structured hexahedral grids (the paper's uniform meshes, Fig. 1
// L617-621) stored in lexicographic order (axis 0 fastest), axis-0 and axis-1
// sides specular, axis-2 sides isothermal or specular (each side uniform).
//
// Same update as flux_kernel (Eq. 3/5 with the Eq. 6 ghosts, L269-292,
// L546-576), organised for the bulk-copy tensor engine:
//  * a CTA owns a tile of 32 x 8 cells (axes 0, 1) and a range of L layers
//    along axis 2, and marches through the layers in the upwind order of the
//    direction, so the axis-2 upwind value of layer z is the previous layer's
//    staged box (no reload);
//  * one stage = the 4 directions of an orbit {d, m0(d), m1(d), m0 m1(d)} under
//    the axis-0 / axis-1 mirrors, each a (32+2) x (8+1) box of I^n (own cells
//    plus the upwind halo row/column), and the I0 row of the layer.  The
//    specular ghost of an axis-0/1 wall face, I^n[b][m(d)][c] (Eq. 6 at the old
//    level), is then the own value of the partner slot in the same stage: no
//    global load and no boundary branch.  The axis-2 ghost layer is a tensor
//    copy too: the isothermal side table I0_b(T_wall) or, for a specular side,
//    the wall layer of the z-mirrored direction;
//  * a producer warp issues every copy (cp.async.bulk.tensor, mbarrier
//    complete_tx) S stages ahead; results go to shared memory and leave with
//    tensor stores; the per-cell energy partial sum_b c_b sum_d w_d I'
//    (L412-418) accumulates in shared memory per layer.
// HBM-bound, 16 B per update; every other byte is an L2 hit (halo boxes,
// I0 rows, the ghost layer).
constexpr int kBoxTX = 32, kBoxTY = 8;
constexpr int kBoxBX = kBoxTX + 2;           // staged box row (own cells + 2: 16-byte rows)
constexpr int kBoxBY = kBoxTY + 1;           // own rows + the upwind halo row
constexpr int kBoxBoxElems = kBoxBX * kBoxBY;  // 306 doubles copied per plane
constexpr int kBoxPlane = 320;               // doubles per staged plane (128-byte aligned)
constexpr int kBoxCells = kBoxTX * kBoxTY;   // 256 threads compute, one cell each
constexpr int kBoxThreads = kBoxCells + 32;  // + the producer warp
constexpr int kBoxMaxStages = 12;
// How I^{n+1} leaves the box kernel (measured on B200): 3-D grids
// store straight from registers (coalesced st.global.cs, no per-layer CTA
// barrier: C4 sustained flux 7.80 -> 7.53 ms); 2-D grids keep the
// shared-memory tile + tensor store (C3 0.84 -> 0.83 ms).  -DBTE_BOX_TMA_STORE:
// tensor stores everywhere.
template <bool FLAT>
constexpr bool box_tma_store() {
#ifdef BTE_BOX_TMA_STORE
    return true;
#else
    return FLAT;
#endif
}
template <bool FLAT>
constexpr bool box_obuf() { return box_tma_store<FLAT>(); }  // (the shared output tile of the tensor stores)
// Resident CTAs per SM the kernel is compiled for (register cap): 3-D grids 2
// (96 registers, 6 stages of 12 KB plus L x 2 KB of energy rows); 2-D grids 3
// (72 registers, no spills, 4 stages): a 2-D stage is one layer, so CTAs are
// short and more of them per SM hide the per-stage handshake (C3 flux 0.83 ->
// 0.96 of measured HBM, measured on B200; 3-D loses with 3).
constexpr int kBoxMinBlocks3D = 2, kBoxMinBlocks2D = 3;
// doubles per stage: 4 direction planes + the I0 row (+ the two rate rows with
// temperature-dependent relaxation times)
template <bool TD>
constexpr int box_stage_elems() { return 4 * kBoxPlane + (TD ? 3 : 1) * kBoxCells; }

// One orbit of directions under the two in-plane mirrors.  Slot j has
// s_0 > 0 for even j, s_0 < 0 for odd j; s_1 > 0 for j < 2, s_1 < 0 for j >= 2;
// slot j ^ 1 is the axis-0 mirror of slot j, slot j ^ 2 the axis-1 mirror.
struct BoxOrbit {
    int32_t d[4];
    int32_t rz[4];  // axis-2 mirror of d[j] (specular axis-2 sides), else -1
};

struct BoxParams {
    int32_t n0, n1, n2;        // grid extents, axis 0 contiguous (n2: layers of the slab tensor)
    int32_t zlo, nown;         // computed layers [zlo, zlo + nown) of the tensor (a z-slab cell
                               // partition keeps halo layers around them; else 0, n2)
    int32_t tiles0, tiles1;    // 32-cell tiles along axis 0, 8-cell tiles along axis 1
    int32_t L, zranges;        // layers per work item, ranges along axis 2
    int32_t n_orb, orb_chunk, n_chunks;  // orbits, orbits per item, chunks
    int32_t nbl, nbb, n_slices;  // band-rows in this launch, band-rows per item, band batches x chunks
    int32_t band0, slot0;      // rank-local first band-row; first energy slot
    int32_t nc;
    int32_t stages;            // shared-memory ring depth
    int32_t zside[2];          // ghost-axis low / high side (3-D: axis 2; 2-D: axis 1): 0 isothermal, 1 specular
    int32_t rsel_cur, rsel_next;  // temperature-dependent rates: table halves (current, next)
    int32_t rate_r2;           // ... R2 weights rate_next / v_b (else the constant cw)
    double dt;
    double g[3];               // A_f / V_c per axis (uniform grid)
    const BoxOrbit *orb;       // [n_orb]
    const double4 *dirs;       // [nd] {s_0, s_1, s_2, w} in grid axes
    double *part;              // [n_slots][nc] energy partials
    double *pool;              // slab pool (direct stores of I^{n+1}): slab s, direction d, tensor
    int64_t slab_elems;        // cell (x, y, z) at pool[s slab_elems + d ps + (z n1 + y) n0 + x]
    int32_t ps;
    const int32_t *fail;       // != 0: a temperature solve of an earlier step failed -> no-op
    int32_t *halt;             // ... latched here for the rest of the step (block 0)
    int32_t in_slab[kMaxBandsPerLaunch];   // launch-local band-row -> slab of I^n
    int32_t out_slab[kMaxBandsPerLaunch];  // ... slab of I^{n+1}
    double dtit[kMaxBandsPerLaunch];       // dt / tau_b (constant rates)
    double kv[kMaxBandsPerLaunch];         // dt v_b
    double cw[kMaxBandsPerLaunch];         // temperature weight c_b (constant rates)
    double inv_v[kMaxBandsPerLaunch];      // 1 / v_b (R2 weight rate / v_b with rate tables)
};

__device__ __forceinline__ void tma_load_5d(void *dst, const void *tmap, int c0, int c1, int c2, int c3, int c4,
                                            uint64_t *bar) {
    asm volatile(
        "cp.async.bulk.tensor.5d.shared::cluster.global.tile.mbarrier::complete_tx::bytes"
        " [%0], [%1, {%2, %3, %4, %5, %6}], [%7];" ::"r"(smem_u32(dst)),
        "l"(reinterpret_cast<uint64_t>(tmap)), "r"(c0), "r"(c1), "r"(c2), "r"(c3), "r"(c4), "r"(smem_u32(bar))
        : "memory");
}
__device__ __forceinline__ void tma_load_3d(void *dst, const void *tmap, int c0, int c1, int c2, uint64_t *bar) {
    asm volatile(
        "cp.async.bulk.tensor.3d.shared::cluster.global.tile.mbarrier::complete_tx::bytes"
        " [%0], [%1, {%2, %3, %4}], [%5];" ::"r"(smem_u32(dst)),
        "l"(reinterpret_cast<uint64_t>(tmap)), "r"(c0), "r"(c1), "r"(c2), "r"(smem_u32(bar))
        : "memory");
}
__device__ __forceinline__ void tma_load_4d(void *dst, const void *tmap, int c0, int c1, int c2, int c3,
                                            uint64_t *bar) {
    asm volatile(
        "cp.async.bulk.tensor.4d.shared::cluster.global.tile.mbarrier::complete_tx::bytes"
        " [%0], [%1, {%2, %3, %4, %5}], [%6];" ::"r"(smem_u32(dst)),
        "l"(reinterpret_cast<uint64_t>(tmap)), "r"(c0), "r"(c1), "r"(c2), "r"(c3), "r"(smem_u32(bar))
        : "memory");
}
__device__ __forceinline__ void tma_store_5d(const void *tmap, const void *src, int c0, int c1, int c2, int c3,
                                             int c4) {
#ifndef BTE_BOX_STORE_NO_HINT
    uint64_t pol;  // I^{n+1} is not read again this step: keep L2 for the halo boxes (C5 +1.7 %)
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
    asm volatile(
        "cp.async.bulk.tensor.5d.global.shared::cta.tile.bulk_group.L2::cache_hint [%0, {%2, %3, %4, %5, %6}], [%1], "
        "%7;" ::"l"(reinterpret_cast<uint64_t>(tmap)),
        "r"(smem_u32(src)), "r"(c0), "r"(c1), "r"(c2), "r"(c3), "r"(c4), "l"(pol)
        : "memory");
#else
    asm volatile("cp.async.bulk.tensor.5d.global.shared::cta.tile.bulk_group [%0, {%2, %3, %4, %5, %6}], [%1];" ::"l"(
                     reinterpret_cast<uint64_t>(tmap)),
                 "r"(smem_u32(src)), "r"(c0), "r"(c1), "r"(c2), "r"(c3), "r"(c4)
                 : "memory");
#endif
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_read_all() { asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }
__device__ __forceinline__ void fence_smem_to_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
__device__ __forceinline__ void bar_compute() { asm volatile("bar.sync 1, %0;" ::"n"(kBoxCells) : "memory"); }

// Tensor maps (host-encoded, see bte_create.cu):
//   tm_in   the slab pool as {n0, n1, n2, nd, n_slabs}, box {34, 9, 1, 1, 1}
//   tm_out  same tensor, box {32, 8, 1, 1, 1} (stores)
//   tm_i0   I0 table as {n0, n1, n2, nb_loc}, box {32, 8, 1, 1}
//   tm_side isothermal axis-2 side tables as {n0, n1, 2, nb_loc}, box {34, 9, 1, 1}
//           (2-D: the axis-1 wall rows as {n0, 2, nb_loc}, box {32, 1, 1})
//   tm_rate rate tables 1/tau_b(T) as {n0, n1, n2, nb_loc, 2}, box {32, 8, 1, 1, 1}
// Box origin of slot j: axis 0 at x0 - 2 (s_0 > 0: upwind is x - 1) or x0
// (s_0 < 0: x + 1); axis 1 at y0 - 1 (s_1 > 0) or y0.
__device__ __forceinline__ int box_xs(int j) { return (j & 1) ? 0 : 2; }
__device__ __forceinline__ int box_hy(int j) { return (j & 2) ? 0 : 1; }

// Work item = (band batch x orbit chunk "slice", 32 x 8 x L cell block "tile"),
// tile fastest, one CTA per item: the hardware block scheduler balances the
// SMs (measured better on B200 than persistent CTAs with static or
// counter-based item assignment) and the resident CTAs work on
// neighbouring tiles of the same slice, so their halo boxes are L2 hits.
struct BoxItem {
    int x0, y0, z0, Lc, k0, k1, o0, o1, slice;
};
__device__ __forceinline__ BoxItem box_item(const BoxParams &p, int item) {
    const int n_tiles = p.tiles0 * p.tiles1 * p.zranges;
    BoxItem w;
    w.slice = item / n_tiles;
    int t = item - w.slice * n_tiles;
    const int t0 = t % p.tiles0;
    t /= p.tiles0;
    const int t1 = t % p.tiles1;
    const int zr = t / p.tiles1;
    w.x0 = t0 * kBoxTX;
    w.y0 = t1 * kBoxTY;
    w.z0 = p.zlo + zr * p.L;
    w.Lc = min(p.L, p.zlo + p.nown - w.z0);
    const int chunk = w.slice % p.n_chunks, batch = w.slice / p.n_chunks;
    w.k0 = batch * p.nbb;
    w.k1 = min(p.nbl, w.k0 + p.nbb);
    w.o0 = chunk * p.orb_chunk;
    w.o1 = min(p.n_orb, w.o0 + p.orb_chunk);
    return w;
}

// Per-orbit constants of a CTA's chunk, formed once in the prologue: the four
// direction ids and weights, the axis-2 mirrors, |s . g| per axis (the same
// for the 4 slots) and the marching order along axis 2.
struct BoxOrbitC {
    int32_t d[4], rz[4];
    double w[4];
    double a[3];
    int32_t asc;
    int32_t pad;
};

template <bool TD, bool FLAT>
__global__ void __launch_bounds__(kBoxThreads, FLAT ? kBoxMinBlocks2D : kBoxMinBlocks3D)
flux_box_kernel(const __grid_constant__ BoxParams p, const __grid_constant__ CUtensorMap tm_in,
                const __grid_constant__ CUtensorMap tm_out, const __grid_constant__ CUtensorMap tm_i0,
                const __grid_constant__ CUtensorMap tm_side, const __grid_constant__ CUtensorMap tm_rate) {
    constexpr int kGhost = box_stage_elems<TD>();  // 2-D: stage offset of the two wall rows
    constexpr int kStage = kGhost + (FLAT ? 2 * kBoxTX : 0);
    constexpr bool flat = FLAT;
    extern __shared__ __align__(128) double bsm[];
#ifdef BTE_BOX_FIXED_S
    constexpr int S = BTE_BOX_FIXED_S;
#else
    const int S = p.stages;
#endif
    double *ring = bsm;                          // [S][kStage]
    constexpr bool kTmaStore = box_tma_store<FLAT>();
    double *obuf = ring + S * kStage;                           // [2][4][256] (tensor stores)
    double *eacc = obuf + (box_obuf<FLAT>() ? 2 * 4 * kBoxCells : 0);  // [L][256]
    BoxOrbitC *sorb = reinterpret_cast<BoxOrbitC *>(eacc + p.L * kBoxCells);  // [orb_chunk]
    __shared__ __align__(8) uint64_t full[kBoxMaxStages];
    __shared__ __align__(8) uint64_t empty[kBoxMaxStages];

    const int tid = threadIdx.x;
    if (flux_halted(p.fail, p.halt)) return;  // (a failed solve earlier in this bte_step call)
    const BoxItem w = box_item(p, blockIdx.x);
    if (tid == 0) {
        for (int s = 0; s < S; ++s) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], kBoxCells / 32);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    for (int i = tid; i < w.o1 - w.o0; i += kBoxThreads) {
        const BoxOrbit ob = p.orb[w.o0 + i];
        BoxOrbitC c;
        for (int q = 0; q < 4; ++q) {
            c.d[q] = ob.d[q];
            c.rz[q] = ob.rz[q];
            c.w[q] = load_dir(p.dirs, ob.d[q]).w;
        }
        const double4 s0 = load_dir(p.dirs, ob.d[0]);
        c.a[0] = fabs(s0.x * p.g[0]);
        c.a[1] = fabs(s0.y * p.g[1]);
        c.a[2] = fabs(s0.z * p.g[2]);
        c.asc = s0.z >= 0.0;
        c.pad = 0;
        sorb[i] = c;
    }
    __syncthreads();

    if (tid >= kBoxCells) {  // ------------------------------------------- producer warp
        if (tid == kBoxCells) {
            int s = 0;
            uint32_t ph = 0, wrapped = 0;  // ring slot, its use parity, ring wrapped once
            for (int k = w.k0; k < w.k1; ++k) {
                const int slab = p.in_slab[k], bl = p.band0 + k;
                for (int o = w.o0; o < w.o1; ++o) {
                    const BoxOrbitC &ob = sorb[o - w.o0];
                    const bool asc = ob.asc;
                    for (int j = flat ? 1 : 0; j <= w.Lc; ++j) {
                        if (wrapped)
                            while (!mbar_try_wait(&empty[s], ph ^ 1u)) {
                            }
                        double *st = ring + s * kStage;
                        if (j == 0) {  // the upwind layer of the range: neighbour range or ghost layer
                            const int zh = asc ? w.z0 - 1 : w.z0 + w.Lc;
                            mbar_arrive_expect_tx(&full[s], 4 * kBoxBoxElems * sizeof(double));
                            for (int q = 0; q < 4; ++q) {
                                const int xs = w.x0 - box_xs(q), ys = w.y0 - box_hy(q);
                                if (zh >= 0 && zh < p.n2)
                                    tma_load_5d(st + q * kBoxPlane, &tm_in, xs, ys, zh, ob.d[q], slab, &full[s]);
                                else if (p.zside[asc ? 0 : 1] == 0)  // isothermal: I0_b(T_wall) side table
                                    tma_load_4d(st + q * kBoxPlane, &tm_side, xs, ys, asc ? 0 : 1, bl, &full[s]);
                                else  // specular: the wall layer of the z-mirrored direction (old level)
                                    tma_load_5d(st + q * kBoxPlane, &tm_in, xs, ys, asc ? 0 : p.n2 - 1, ob.rz[q],
                                                slab, &full[s]);
                            }
                        } else {
                            const int z = asc ? w.z0 + j - 1 : w.z0 + w.Lc - j;
                            // 2-D: the isothermal wall rows I0_b(T_wall) of the tiles on those walls (Eq. 6)
                            const bool glo = flat && p.zside[0] == 0 && w.y0 == 0;
                            const bool ghi = flat && p.zside[1] == 0 && w.y0 + kBoxTY >= p.n1;
                            mbar_arrive_expect_tx(&full[s], (4 * kBoxBoxElems + (TD ? 3 : 1) * kBoxCells +
                                                             (glo + ghi) * kBoxTX) * sizeof(double));
                            if (glo) tma_load_3d(st + kGhost, &tm_side, w.x0, 0, bl, &full[s]);
                            if (ghi) tma_load_3d(st + kGhost + kBoxTX, &tm_side, w.x0, 1, bl, &full[s]);
                            for (int q = 0; q < 4; ++q)
                                tma_load_5d(st + q * kBoxPlane, &tm_in, w.x0 - box_xs(q), w.y0 - box_hy(q), z,
                                            ob.d[q], slab, &full[s]);
                            tma_load_4d(st + 4 * kBoxPlane, &tm_i0, w.x0, w.y0, z - p.zlo, bl, &full[s]);
                            if (TD) {
                                tma_load_5d(st + 4 * kBoxPlane + kBoxCells, &tm_rate, w.x0, w.y0, z - p.zlo, bl,
                                            p.rsel_cur, &full[s]);
                                tma_load_5d(st + 4 * kBoxPlane + 2 * kBoxCells, &tm_rate, w.x0, w.y0, z - p.zlo, bl,
                                            p.rsel_next, &full[s]);
                            }
                        }
                        if (++s == S) {
                            s = 0;
                            ph ^= 1u;
                            wrapped = 1;
                        }
                    }
                }
            }
        }
        return;
    }

    // ------------------------------------------------------------------ compute warps
    const int tx = tid & 31, ty = tid >> 5, lane = tid & 31;
    const int gx = w.x0 + tx, gy = w.y0 + ty;
    const bool valid = gx < p.n0 && gy < p.n1;
    // staged-plane offsets of this thread: own value, axis-0 and axis-1 upwind
    // values per slot (walls: the mirrored slot's own value, Eq. 6 specular)
    int own[4], ux[4], uy[4];
#pragma unroll
    for (int q = 0; q < 4; ++q) own[q] = q * kBoxPlane + (ty + box_hy(q)) * kBoxBX + tx + box_xs(q);
#pragma unroll
    for (int q = 0; q < 4; ++q) {
        const bool wall0 = (q & 1) ? gx == p.n0 - 1 : gx == 0;
        const bool wall1 = (q & 2) ? gy == p.n1 - 1 : gy == 0;
        ux[q] = wall0 ? own[q ^ 1] : own[q] + ((q & 1) ? 1 : -1);
        uy[q] = wall1 ? own[q ^ 2] : own[q] + ((q & 2) ? kBoxBX : -kBoxBX);
        if (flat && wall1 && p.zside[(q & 2) ? 1 : 0] == 0) uy[q] = kGhost + ((q & 2) ? kBoxTX : 0) + tx;
    }
    for (int l = 0; l < w.Lc; ++l) eacc[l * kBoxCells + tid] = 0.0;
    // byte offsets of the staged values inside a stage (one add per shared load)
    uint32_t own_b[4], ux_b[4], uy_b[4];
#pragma unroll
    for (int q = 0; q < 4; ++q) {
        own_b[q] = (uint32_t)own[q] * 8u;
        ux_b[q] = (uint32_t)ux[q] * 8u;
        uy_b[q] = (uint32_t)uy[q] * 8u;
        // (keep the byte offsets in registers: the loads then address [offset + stage base])
        asm volatile("" : "+r"(own_b[q]), "+r"(ux_b[q]), "+r"(uy_b[q]));
    }
    // direct stores: a warp's 32 cells are one 256-byte row of a plane
    const int32_t plane = p.n0 * p.n1;
    const int32_t cell_off = gy * p.n0 + gx;

    int s = 0, sp = 0;
    uint32_t ph = 0, ob = 0;
    double pv[4] = {0.0, 0.0, 0.0, 0.0};  // the previous layer's own values: this layer's axis-2 upwind values
    for (int k = w.k0; k < w.k1; ++k) {
        const double kv = p.kv[k], dtit_k = p.dtit[k], cw_k = p.cw[k];  // (per band-row, once)
        double *const oslab = p.pool + (int64_t)p.out_slab[k] * p.slab_elems + cell_off;
        for (int o = w.o0; o < w.o1; ++o) {
            const BoxOrbitC &orb = sorb[o - w.o0];
            const bool asc = orb.asc;
            double wq[4];
#pragma unroll
            for (int q = 0; q < 4; ++q) wq[q] = orb.w[q];
            const double kvout = kv * ((orb.a[0] + orb.a[1]) + orb.a[2]);
            const double coef_c = (1.0 - dtit_k) - kvout;  // constant rates
            const double m0 = -orb.a[0], m1 = -orb.a[1], m2 = -orb.a[2];
            // output pointers of the orbit's 4 directions at the first computed layer; they
            // move one plane per layer in the marching direction (slab_elems < 2^31)
            double *op[4];
            const int32_t zfirst = asc ? w.z0 : w.z0 + w.Lc - 1;
            const int64_t dz = asc ? plane : -(int64_t)plane;
#pragma unroll
            for (int q = 0; q < 4; ++q) op[q] = oslab + (orb.d[q] * p.ps + zfirst * plane);
            for (int j = flat ? 1 : 0; j <= w.Lc; ++j) {
                while (!mbar_try_wait(&full[s], ph)) {
                }
                const char *const cb = reinterpret_cast<const char *>(ring + s * kStage);  // this stage
                auto at = [cb](uint32_t b) { return *reinterpret_cast<const double *>(cb + b); };
                if (j == 0) {  // the range's upwind layer: its values to registers
#pragma unroll
                    for (int q = 0; q < 4; ++q) pv[q] = at(own_b[q]);
                    sp = s;
                } else {
                    const int z = asc ? w.z0 + j - 1 : w.z0 + w.Lc - j;
                    const double *cur = ring + s * kStage;
                    double dtit, coef, cw;
                    if (TD) {  // 1/tau_b of this cell at the rate temperature; R2 weight at the next one
                        dtit = p.dt * cur[4 * kBoxPlane + kBoxCells + tid];
                        coef = (1.0 - dtit) - kvout;
                        cw = p.rate_r2 ? cur[4 * kBoxPlane + 2 * kBoxCells + tid] * p.inv_v[k] : cw_k;
                    } else {
                        dtit = dtit_k;
                        coef = coef_c;
                        cw = cw_k;
                    }
                    const double src = dtit * cur[4 * kBoxPlane + tid];
                    double *out = obuf + ob * (4 * kBoxCells);  // (tensor stores)
                    double acc = 0.0;
#pragma unroll
                    for (int q = 0; q < 4; ++q) {
                        const double ic = at(own_b[q]);
                        double infl = m0 * at(ux_b[q]);
                        infl = fma(m1, at(uy_b[q]), infl);
                        if (!flat) infl = fma(m2, pv[q], infl);
                        pv[q] = ic;  // (the next layer's axis-2 upwind value)
                        const double inew = fma(ic, coef, fma(-kv, infl, src));
                        if constexpr (kTmaStore) {
                            out[q * kBoxCells + tid] = inew;
                        } else {
                            if (valid) __stcs(op[q], inew);
                            op[q] += dz;
                        }
                        acc = fma(wq[q], inew, acc);
                    }
                    double *ea = eacc + (z - w.z0) * kBoxCells + tid;
                    *ea = fma(cw, acc, *ea);
                    __syncwarp();
                    // release the previous layer's stage now (one layer late: keeps the producer
                    // from running further ahead, which measured more DRAM re-reads of halo boxes)
                    if (lane == 0) {
                        if (flat) {
                            mbar_arrive(&empty[s]);
                        } else {
                            mbar_arrive(&empty[sp]);
                            if (j == w.Lc) mbar_arrive(&empty[s]);
                        }
                    }
                    sp = s;
                    if constexpr (kTmaStore) {
                        fence_smem_to_async();
                        if (tid == 0) bulk_wait_read_all();  // the other output buffer has been read
                        bar_compute();
                        if (tid == 0) {
#pragma unroll
                            for (int q = 0; q < 4; ++q)
                                tma_store_5d(&tm_out, out + q * kBoxCells, w.x0, w.y0, z, orb.d[q], p.out_slab[k]);
                            bulk_commit();
                        }
                        ob ^= 1u;
                    }
                }
                if (++s == S) {
                    s = 0;
                    ph ^= 1u;
                }
            }
        }
    }
    if (valid) {
        double *part = p.part + (int64_t)(p.slot0 + w.slice) * p.nc;
        for (int l = 0; l < w.Lc; ++l)
            part[((int64_t)(w.z0 - p.zlo + l) * p.n1 + gy) * p.n0 + gx] = eacc[l * kBoxCells + tid];
    }
    if (kTmaStore && tid == 0) bulk_wait_all();
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
    // an iterate T is accepted when its Newton correction |g / g'| <= racc T,
    // racc = max(rtol / 100, 16 eps): it then lies within ~rtol / 100 of the root
    // the oracle's |dT| <= rtol T test converges to (reading 25); rtol
    // bounds the bisection safeguard's bracket
    double W, rtol, racc;
    int32_t maxit;
    int32_t *iter_max;
    int32_t *fail;
    // temperature-dependent relaxation times (N1): 1/tau_b(T) = ra + rb T exp(-rth / T)
    int32_t td;            // 0: constant rates (cw); 1: rate law
    int32_t tr_step;       // 1: a step's solve (rate temperature <- T^n, weights at T^n); 0: weights at Tr
    int32_t tr_now;        // rates of the current T (reading 26): the rate temperature follows T
    int32_t r2;            // R2 weights rate / v_b (else R1 cw = 1 / v_b)
    const double *ra, *rb, *rth, *inv_v;  // [nb] global
    double *Tr;            // [nc] rate temperature
    double *rate_out;      // [nb_loc][nc] rates of the local rows at the new T
    int32_t single;        // R3: one linearised first-law step, no convergence test (N4)
    double *T_out;         // diagnostic / chunk solve: write T here only (state untouched)
    int32_t c_lo;          // chunk solve: cells [c_lo, c_lo + nc) of the mesh, E indexed from c_lo
    int32_t neg_fail;      // chunk solve: a failed cell writes -T^n (decoded by newton_finish_kernel)
    // ENOCONV stop (a step's solve): halt = the flux launch's latch (a solve of an
    // earlier step of the call failed: no-op); done != nullptr: this launch ends
    // the step and block 0 counts it
    const int32_t *halt;
    int32_t *done;
    // the I0 table of ALL band-rows at the starting temperature T0 = T[c]
    // ([nb][nc_tab], the previous step's refresh; nullptr when this rank holds
    // only some rows): the first g / g' evaluation of a solve reads it instead
    // of nb expm1 (I0 = C / expm1(x), 1 / expm1(x) = I0 / C)
    const double *i0_t0;
    int32_t nc_tab;
    // terms of the temperature equation with constant weights (see Terms; 0: per row)
    int32_t n_terms;
    const double *t_th, *t_k, *t_ic;
    const int32_t *t_rep;
    const int32_t *t_nrow;  // [nb] the next row of the same term (-1: none)
    // spec != 0 (this rank holds every row, whole-mesh solve): an evaluation of g at
    // an iterate T_k also stores I0_b(T_k) = C_b q (the I0 refresh), so a solve that
    // accepts T_k needs no refresh of its own; fresh[c] (step solves into T_out)
    // tells newton_finish_kernel that cell c's rows are stored already
    int32_t spec;
    int8_t *fresh;
};

// 1/tau_b(T) of the rate law (N1, L666-669): impurity-like + Umklapp-like terms.
__device__ __forceinline__ double tau_rate(double a, double b, double th, double T) {
    return a + b * T * exp(-th / T);
}

struct Gsum { double g, gp; };

// The temperature equation g(T) = W sum_j K_j I0(theta_j; T) / C_j - E as a sum
// of TERMS j: with constant weights the rows that share theta (the LA and TA
// rows of a band: 55 rows, 40 terms for the paper's 40 bands) are one term,
// K_j = sum_{b in j} c_b C_b, so one expm1 serves them (bte_create builds the
// terms); with the rate law under R2 the weights depend on the cell, and the
// terms are the rows, K_b = rate_b(Tw) / v_b C_b.  With q = 1 / expm1(x),
// x = theta / T: I0 = C q, dI0/dT = I0 (x / T) (1 + q).
struct Terms {
    const double *th, *k, *ic;  // per term: theta_j, K_j (nullptr: per row, c_b C_b), 1 / C of its representative
    const int32_t *rep;          // representative row (nullptr: the row itself)
    const int32_t *nrow;         // the next row of the same term (with rep)
    int n;
    bool law;                    // per-cell weights: K_b = tau_rate(a, b, th, Tw) iv_b C_b
    const double *C, *w, *ra, *rb, *rth, *iv;
    double Tw;
    __device__ __forceinline__ double K(int j) const {
        return law ? tau_rate(ra[j], rb[j], rth[j], Tw) * iv[j] * C[j] : k ? k[j] : w[j] * C[j];
    }
    __device__ __forceinline__ int row(int j) const { return rep ? rep[j] : j; }
};

// Shared-memory band / term tables of the solve kernels (newton_smem on the host):
// 8 row arrays [nb] (C, theta, c, rate a / b / theta, 1 / v, 1 / C), then 3 term
// arrays [n_terms] (theta, K, 1 / C of the representative) and the int32 term
// representatives.
struct SolveTables {
    double *C, *th, *w, *a, *b, *r, *v, *ic, *tth, *tk, *tic;
    int32_t *trep, *nrow;
};
__device__ __forceinline__ SolveTables solve_tables(double *sm, int nb, int nt) {
    SolveTables t;
    t.C = sm; t.th = sm + nb; t.w = sm + 2 * nb; t.a = sm + 3 * nb; t.b = sm + 4 * nb;
    t.r = sm + 5 * nb; t.v = sm + 6 * nb; t.ic = sm + 7 * nb;
    t.tth = sm + 8 * nb; t.tk = t.tth + nt; t.tic = t.tk + nt;
    t.trep = reinterpret_cast<int32_t *>(t.tic + nt);
    t.nrow = reinterpret_cast<int32_t *>(t.tic + 2 * nt);  // (after the nt doubles holding trep)
    return t;
}
__device__ __forceinline__ void load_solve_tables(const SolveTables &t, const NewtonParams &p) {
    for (int b = threadIdx.x; b < p.nb; b += blockDim.x) {
        t.ic[b] = 1.0 / p.Cb[b];
        t.C[b] = p.Cb[b];
        t.th[b] = p.theta[b];
        t.w[b] = p.cw[b];
        if (p.td) {
            t.a[b] = p.ra[b];
            t.b[b] = p.rb[b];
            t.r[b] = p.rth[b];
            t.v[b] = p.inv_v[b];
        }
    }
    for (int j = threadIdx.x; j < p.n_terms; j += blockDim.x) {
        t.tth[j] = p.t_th[j];
        t.tk[j] = p.t_k[j];
        t.tic[j] = p.t_ic[j];
        t.trep[j] = p.t_rep[j];
    }
    if (p.t_nrow)
        for (int b = threadIdx.x; b < p.nb; b += blockDim.x) t.nrow[b] = p.t_nrow[b];
}
// The terms of a cell's solve (Tw: the rate temperature of its weights).
__device__ __forceinline__ Terms solve_terms(const SolveTables &t, const NewtonParams &p, double Tw) {
    Terms q;
    q.law = p.td && p.r2;
    const bool terms = !q.law && p.n_terms > 0;  // (else one term per row: the rate law, or other weights)
    q.th = terms ? t.tth : t.th;
    q.k = terms ? t.tk : nullptr;
    q.ic = terms ? t.tic : t.ic;
    q.rep = terms ? t.trep : nullptr;
    q.nrow = t.nrow;
    q.n = terms ? p.n_terms : p.nb;
    q.C = t.C; q.w = t.w; q.ra = t.a; q.rb = t.b; q.rth = t.r; q.iv = t.v;
    q.Tw = Tw;
    return q;
}

__device__ __forceinline__ Gsum g_eval(const Terms &t, double W, double E, double T) {
    double g = 0.0, gp = 0.0;
    const double it = 1.0 / T;
    for (int j = 0; j < t.n; ++j) {
        const double x = t.th[j] * it;
        const double q = 1.0 / expm1(x);
        const double kq = t.K(j) * q;
        g += kq;
        gp = fma(kq, (x * it) * (1.0 + q), gp);
    }
    return {W * g - E, W * gp};
}

// g, g' at T0 from the stored table i0_t0[b][c] = I0_b(T0) (q = I0 / C).
__device__ __forceinline__ Gsum g_eval_table(const Terms &t, double W, double E, double T0, const double *i0_t0,
                                             int64_t stride) {
    double g = 0.0, gp = 0.0;
    const double it = 1.0 / T0;
    for (int j = 0; j < t.n; ++j) {
        const double x = t.th[j] * it;
        const double q = __ldg(i0_t0 + t.row(j) * stride) * t.ic[j];
        const double kq = t.K(j) * q;
        g += kq;
        gp = fma(kq, (x * it) * (1.0 + q), gp);
    }
    return {W * g - E, W * gp};
}

__device__ __forceinline__ double g_only(const Terms &t, double W, double E, double T) {
    double g = 0.0;
    for (int j = 0; j < t.n; ++j) g += t.K(j) / expm1(t.th[j] / T);
    return W * g - E;
}

// g and its first three T-derivatives.  Per term, with q = 1 / expm1(x), x = theta / T,
// s = q (1 + q), m = (1 + 2 q) x:  d/dT q = s x / T,  d2 = s x (m - 2) / T^2,
// d3 = s x (m^2 - 6 m + 6 + 2 s x^2) / T^3 (no further exponentials: the
// Householder step below costs a few FMAs per term on top of Newton's).
struct Gder { double g, g1, g2, g3; };
__device__ __forceinline__ void der_term(double K, double q, double x, double &a0, double &a1, double &a2,
                                         double &a3) {
    const double sx = q * (1.0 + q) * x, m = fma(2.0 * q, x, x);
    const double ks = K * sx;
    a0 = fma(K, q, a0);
    a1 += ks;
    a2 = fma(ks, m - 2.0, a2);
    a3 = fma(ks, fma(m, m - 6.0, 6.0) + 2.0 * sx * x, a3);
}
__device__ __forceinline__ Gder der_finish(double W, double E, double T, double a0, double a1, double a2, double a3) {
    const double it = 1.0 / T;
    return {W * a0 - E, W * a1 * it, W * a2 * it * it, W * a3 * it * it * it};
}
// The correction h (T <- T - h) of Householder's third-order method (convergence
// order 4): one step from the previous step's I0 table reaches |h| <= rtol T at
// the next evaluation for the per-step temperature changes of an explicit step
// (~1e-4 T), so a solve takes that one evaluation.  Newton's correction where the
// higher-order one is not finite or strays from it (far from the root).
__device__ __forceinline__ double householder_step(const Gder &d) {
    const double newton = d.g / d.g1;
    const double num = 3.0 * d.g * (2.0 * d.g1 * d.g1 - d.g * d.g2);
    const double den = 6.0 * d.g1 * d.g1 * d.g1 - 6.0 * d.g * d.g1 * d.g2 + d.g * d.g * d.g3;
    const double h = num / den;
    return (isfinite(h) && fabs(h - newton) <= 0.5 * fabs(newton)) ? h : newton;
}
// I0 of the rows of term j at the iterate (q = 1 / expm1(theta_j / T)): the
// speculative refresh of an evaluation (NewtonParams::spec), local rows only.
__device__ __forceinline__ void store_term_rows(const Terms &t, const SolveTables &tb, const NewtonParams &p, int j,
                                                double q, int c) {
    for (int b = t.row(j); b >= 0; b = t.rep ? t.nrow[b] : -1) {
        const int k = b - p.b_lo;
        if (k >= 0 && k < p.nb_loc) p.i0[(size_t)k * p.nc + c] = tb.C[b] * q;
    }
}
// One evaluation of g, g', g'', g''' at T: from the stored I0 table (tab: I0 at T,
// q = I0 / C) or with one expm1 per term, storing the rows' I0 (store).  The
// table loads go in batches of 8 issued together (one thread per cell: 40
// dependent loads otherwise bound the solve, ncu C4); the sums run in term order.
constexpr int kTermBatch = 8;
__device__ __forceinline__ Gder g_eval_der(const Terms &t, const SolveTables &tb, const NewtonParams &p, double E,
                                           double T, const double *tab, int64_t stride, bool store, int c) {
    double a0 = 0.0, a1 = 0.0, a2 = 0.0, a3 = 0.0;
    const double it = 1.0 / T;
    if (tab) {
        for (int j0 = 0; j0 < t.n; j0 += kTermBatch) {
            double qv[kTermBatch];
#pragma unroll
            for (int u = 0; u < kTermBatch; ++u)
                qv[u] = __ldg(tab + t.row(min(j0 + u, t.n - 1)) * stride);  // (a clamped duplicate is not summed)
#pragma unroll
            for (int u = 0; u < kTermBatch; ++u) {
                const int j = j0 + u;
                if (j < t.n) der_term(t.K(j), qv[u] * t.ic[j], t.th[j] * it, a0, a1, a2, a3);
            }
        }
    } else {
        for (int j = 0; j < t.n; ++j) {
            const double x = t.th[j] * it;
            const double q = 1.0 / expm1(x);
            if (store) store_term_rows(t, tb, p, j, q, c);
            der_term(t.K(j), q, x, a0, a1, a2, a3);
        }
    }
    return der_finish(p.W, E, T, a0, a1, a2, a3);
}

__global__ void __launch_bounds__(128, 8) newton_kernel(const __grid_constant__ NewtonParams p);

// ---------------------------------------------------------------------------
// The same per-cell temperature solve with a GROUP of G lanes per cell (the
// step's solve on small meshes): lane l of the group evaluates terms l, l + G,
// ... and butterfly shuffles inside the group give every lane bitwise the same
// sums (each level adds a commutative pair), so the Newton iterates and the
// bisection safeguard are group-uniform.  A cell's terms x ~3 iterations of
// expm1 are spread over G lanes: small meshes (C3: 14,400 cells, G = 32) fill
// the GPU instead of a few warps per SM.  Output: T_out[c] = T^{n+1} (or -T^n
// on failure); the epilogue (T, Tr, I0, rates) is newton_finish_kernel's.
template <int G>
__device__ __forceinline__ double group_sum(double v, unsigned mask) {
#pragma unroll
    for (int off = G / 2; off > 0; off >>= 1) v += __shfl_xor_sync(mask, v, off);
    return v;
}

// R = terms per lane (ceil(n / G) rounded up to a power of two; the per-lane
// coefficients K stay in registers).
template <int G, int R>
__device__ __forceinline__ Gsum g_eval_group(const Terms &t, const double *kl, double W, double E, double T, int lane,
                                             unsigned mask, const double *tab, int64_t stride) {
    double g = 0.0, gp = 0.0;
    const double it = 1.0 / T;
#pragma unroll
    for (int r = 0; r < R; ++r) {
        const int j = lane + G * r;
        if (j < t.n) {
            const double x = t.th[j] * it;
            const double q = tab ? __ldg(tab + t.row(j) * stride) * t.ic[j] : 1.0 / expm1(x);
            const double kq = kl[r] * q;
            g += kq;
            gp = fma(kq, (x * it) * (1.0 + q), gp);
        }
    }
    return {W * group_sum<G>(g, mask) - E, W * group_sum<G>(gp, mask)};
}

template <int G, int R>
__device__ __forceinline__ double g_only_group(const Terms &t, const double *kl, double W, double E, double T,
                                               int lane, unsigned mask) {
    double g = 0.0;
#pragma unroll
    for (int r = 0; r < R; ++r) {
        const int j = lane + G * r;
        if (j < t.n) g += kl[r] / expm1(t.th[j] / T);
    }
    return W * group_sum<G>(g, mask) - E;
}

constexpr int kSumSlotWarps = 8;  // sum_slots_kernel: warps per 32 cells

template <int G, int R>
__device__ __forceinline__ Gder g_eval_der_group(const Terms &t, const SolveTables &tb, const NewtonParams &p,
                                                 const double *kl, double E, double T, int lane, unsigned mask,
                                                 const double *tab, int64_t stride, bool store, int c) {
    double a0 = 0.0, a1 = 0.0, a2 = 0.0, a3 = 0.0;
    const double it = 1.0 / T;
#pragma unroll
    for (int r = 0; r < R; ++r) {
        const int j = lane + G * r;
        if (j < t.n) {
            const double x = t.th[j] * it;
            const double q = tab ? __ldg(tab + t.row(j) * stride) * t.ic[j] : 1.0 / expm1(x);
            if (store) store_term_rows(t, tb, p, j, q, c);
            der_term(kl[r], q, x, a0, a1, a2, a3);
        }
    }
    return der_finish(p.W, E, T, group_sum<G>(a0, mask), group_sum<G>(a1, mask), group_sum<G>(a2, mask),
                      group_sum<G>(a3, mask));
}

template <int G, int R>
__global__ void newton_lanes_kernel(const __grid_constant__ NewtonParams p) {
    if (p.halt && *p.halt) return;
    if (p.done && blockIdx.x == 0 && threadIdx.x == 0) atomicAdd(p.done, 1);  // (the step's last kernel)
    extern __shared__ double sm[];
    const SolveTables tb = solve_tables(sm, p.nb, p.n_terms);
    load_solve_tables(tb, p);
    __syncthreads();
    const int lane = threadIdx.x & (G - 1);
    const unsigned mask = G == 32 ? 0xffffffffu : ((1u << G) - 1u) << ((threadIdx.x & 31) & ~(G - 1));
    const int cl = (blockIdx.x * blockDim.x + threadIdx.x) / G;  // chunk-local cell
    if (cl >= p.nc) return;  // (whole groups)
    const int c = p.c_lo + cl;
    double E;
    if (p.E) {
        E = p.E[cl];
    } else {  // the slot sum in sum_slots_kernel's order, bit for bit: lane w < 8 sums slots
              // w, w + 8, ...; the partials are then added in lane order (G >= 8)
        double e = 0.0;
        if (lane < kSumSlotWarps) {
            int s = lane;
            for (; s + 3 * kSumSlotWarps < p.n_slots; s += 4 * kSumSlotWarps) {
                double v[4];
#pragma unroll
                for (int u = 0; u < 4; ++u) v[u] = __ldcs(p.part + (size_t)(s + u * kSumSlotWarps) * p.nc + c);
#pragma unroll
                for (int u = 0; u < 4; ++u) e += v[u];
            }
            for (; s < p.n_slots; s += kSumSlotWarps) e += __ldcs(p.part + (size_t)s * p.nc + c);
        }
        const int base = (threadIdx.x & 31) & ~(G - 1);  // the group's first lane in the warp
        E = __shfl_sync(mask, e, base);
#pragma unroll
        for (int k = 1; k < kSumSlotWarps; ++k) E += __shfl_sync(mask, e, base + k);
    }
    const double T0 = p.T[c];
    const Terms t = solve_terms(tb, p, p.td ? (p.tr_step ? T0 : p.Tr[c]) : 0.0);  // a step: weights at T^n
    double kl[R];
#pragma unroll
    for (int r = 0; r < R; ++r) {
        const int j = lane + G * r;
        kl[r] = j < t.n ? t.K(j) : 0.0;
    }
    const double *tab = p.i0_t0 ? p.i0_t0 + c : nullptr;  // (I0 at T0 of every row)
    double T = T0;
    bool ok = false, fresh = false;
    int it = 0;
    if (E > 0.0 && isfinite(E) && p.single) {  // R3: T + (E - E_eq(T)) / C(T)
        const Gsum gs = g_eval_group<G, R>(t, kl, p.W, E, T, lane, mask, tab, p.nc_tab);
        const double Tn = T - gs.g / gs.gp;
        it = 1;
        if (Tn > 0.0 && isfinite(Tn)) {
            T = Tn;
            ok = true;
        }
    } else if (E > 0.0 && isfinite(E)) {  // (newton_kernel's iteration, the sums over the group)
        for (it = 1; it <= p.maxit; ++it) {
            const bool from_tab = it == 1 && tab, store = p.spec && !from_tab;
            const Gder d = g_eval_der_group<G, R>(t, tb, p, kl, E, T, lane, mask, from_tab ? tab : nullptr, p.nc_tab,
                                                  store, c);
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
            for (int k = 0; k < 2000 && g_only_group<G, R>(t, kl, p.W, E, lo, lane, mask) > 0.0; ++k) lo *= 0.5;
            for (int k = 0; k < 2000 && g_only_group<G, R>(t, kl, p.W, E, hi, lane, mask) < 0.0; ++k) hi *= 2.0;
            if (g_only_group<G, R>(t, kl, p.W, E, lo, lane, mask) <= 0.0 &&
                g_only_group<G, R>(t, kl, p.W, E, hi, lane, mask) >= 0.0) {
                for (int k = 0; k < 400 && (hi - lo) > p.rtol * hi; ++k) {
                    const double mid = 0.5 * (lo + hi);
                    if (g_only_group<G, R>(t, kl, p.W, E, mid, lane, mask) < 0.0) lo = mid; else hi = mid;
                }
                T = 0.5 * (lo + hi);
                ok = true;
            }
            it = p.maxit + 1;
        }
    }
    if (p.T_out) {  // (chunk solves: newton_finish_kernel completes the step)
        if (lane == 0) {
            if (!ok) atomicExch(p.fail, 1);
            atomicMax(p.iter_max, it);
            p.T_out[c] = ok ? T : (p.neg_fail ? -T0 : T0);
            if (p.fresh) p.fresh[c] = (int8_t)(ok && fresh);
        }
        return;
    }
    // the epilogue of newton_finish_kernel, by the group: T, Tr, and the local rows'
    // I0 (unless stored by the accepting evaluation) and rates at the new T
    if (!ok) T = T0;  // (a failed cell keeps T^n)
    if (lane == 0) {
        if (!ok) atomicExch(p.fail, 1);
        atomicMax(p.iter_max, it);
        if (p.td && (p.tr_now || p.tr_step)) p.Tr[c] = p.tr_now ? T : T0;
        p.T[c] = T;
    }
    const double iT = 1.0 / T;
    for (int k = lane; k < p.nb_loc; k += G) {
        const int b = p.b_lo + k;
        if (!(ok && fresh)) p.i0[(size_t)k * p.nc + c] = tb.C[b] * (1.0 / expm1(tb.th[b] * iT));
        if (p.td) p.rate_out[(size_t)k * p.nc + c] = tau_rate(tb.a[b], tb.b[b], tb.r[b], T);
    }
}

// Band-sharded step, after the all-gather of the chunk solves:
// T^{n+1} for every cell (a negative value marks a failed cell of some rank:
// flag it on every rank and keep T^n), the rate temperature Tr <- T^n, and the
// local rows of I0 and of the rate table at T^{n+1} -- the epilogue of
// newton_kernel, bit for bit.
// One thread per (local row, cell): T, Tr from the k = 0 threads.
__global__ void newton_finish_kernel(const double *__restrict__ Tg, double *__restrict__ T, int nc, int b_lo,
                                     int nb_loc, const double *__restrict__ Cb, const double *__restrict__ theta,
                                     double *__restrict__ i0, int td, const double *__restrict__ ra,
                                     const double *__restrict__ rb, const double *__restrict__ rth,
                                     double *__restrict__ Tr, double *__restrict__ rate_out, int32_t *fail,
                                     const int32_t *__restrict__ halt, int32_t *done, int tr_now,
                                     const int8_t *__restrict__ fresh);

// Rate table of the local rows at temperature T: out[k][c] = 1/tau_{b_lo+k}(T_c).
__global__ void rate_table_kernel(const double *__restrict__ T, int nc, int b_lo, int nb_loc,
                                  const double *__restrict__ ra, const double *__restrict__ rb,
                                  const double *__restrict__ rth, double *__restrict__ out);

// E[c] = sum_s part[s][c]  (world > 1: the local partial, all-reduced afterwards)
__global__ void sum_slots_kernel(const double *__restrict__ part, int n_slots, int nc, double *__restrict__ E,
                                 const int32_t *__restrict__ halt);

// E_loc[c] = sum_{local b} c_b sum_d w_d I[b][d][c] of the current state.
// (rate: R2 with the rate law: c_b = rate[k][c] inv_v[k] at the rate temperature)
__global__ void energy_kernel(const double *__restrict__ pool, const int32_t *__restrict__ slot,
                              int64_t slab_elems, int ps, int nb_loc, int nd, int nc,
                              const double4 *__restrict__ dirs, const double *__restrict__ cw,
                              const double *__restrict__ rate, const double *__restrict__ inv_v,
                              double *__restrict__ E);

// I0 table of the local rows: i0[k][c] = C_{b_lo+k} / expm1(theta / T_c)
__global__ void i0_table_kernel(const double *__restrict__ T, int nc, int b_lo, int nb_loc,
                                const double *__restrict__ Cb, const double *__restrict__ theta,
                                double *__restrict__ i0);

// Equilibrium field I[k][d][c] = i0[k][c] into the current slabs (blockIdx.y = k).
__global__ void equilibrium_kernel(double *__restrict__ pool, const int32_t *__restrict__ slot,
                                   int64_t slab_elems, int ps, int nd, int nc,
                                   const double *__restrict__ i0);

// Isothermal ghost table i0w[k][f] = I0_{b_lo+k}(T_wall(f)) (Eq. 6, constant in time).
__global__ void i0w_kernel(const double *__restrict__ twall, int n_iso, int b_lo, int nb_loc,
                           const double *__restrict__ Cb, const double *__restrict__ theta,
                           double *__restrict__ i0w);

// S_max = max_{c,d} sum_faces max(s_d . g, 0) (positivity bound of the step).
// Paired layout: g holds the "+" face of each pair and the sum is sum |s.g|.
template <int DIM>
__global__ void outflow_max_kernel(int nc, int mf, int paired, int nd, const double *__restrict__ gx,
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
            out += paired ? fabs(a) : fmax(a, 0.0);
        }
        m = fmax(m, out);
    }
    atomicMax(smax_bits, (unsigned long long)__double_as_longlong(m));  // m >= 0: bit order = value order
}

// Isothermal axis-2 side tables of the box kernel: out[k][i] = I0w[k][col[i]]
// (Eq. 6 ghost I0_b(T_wall), already evaluated by i0w_kernel); 0 where no column.
__global__ void side_table_kernel(const double *__restrict__ i0w, int n_iso, const int32_t *__restrict__ col,
                                  int n_side, int nb_loc, double *__restrict__ out);

// dst[r][u] = src[r * stride + pos[u]]  (internal -> caller cell order).
__global__ void gather_rows_kernel(const double *__restrict__ src, const int32_t *__restrict__ pos,
                                   int nc, int64_t stride, int64_t rows, double *__restrict__ dst);

// dst[r * stride + pos[u]] = src[r][u]  (caller -> internal order)
__global__ void scatter_rows_kernel(const double *__restrict__ src, const int32_t *__restrict__ pos,
                                    int nc, int64_t stride, int64_t rows, double *__restrict__ dst);

// ---------------------------------------------------------------------------
// Halo exchange of a cell-partitioned run (the paper's
// cell-parallel split, L728-735, L768-772).  The upwind values a rank reads
// across a cut face are the neighbour part's I^n at the old level, exactly as
// for an interior face (Eq. 3): they live in extra columns
// [nc, nc + n_halo) of every slab, which the flux kernels read like any other
// neighbour column and never write (z-slab partitions of box grids: whole
// halo layers before / after the owned ones).  One segment per neighbour part, layout
// buf[k][j][i] over the local band-rows k, the segment's direction list j and
// its cell list i (only directions that flow across the cut, s_d . n < 0 at
// the reading cell's face).
struct HaloParams {
    double *row[kMaxBandsPerLaunch];  // current slab of local band-row k
    const int32_t *cells;             // column of send cell i (pack) / of halo cell i (unpack)
    const int32_t *dirs;              // direction list of the segment
    int32_t n, n_dirs, nb_loc, ps;
    const int32_t *fail;              // != 0: a solve of an earlier step of the call failed (no-op)
};

__global__ void halo_pack_kernel(const __grid_constant__ HaloParams p, double *__restrict__ buf);

__global__ void halo_unpack_kernel(const __grid_constant__ HaloParams p, const double *__restrict__ buf);

}  // namespace bte
