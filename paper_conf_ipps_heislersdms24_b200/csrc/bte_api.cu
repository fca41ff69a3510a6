// bte_api.cu -- host runtime behind include/bte.h.
//
// Owns validation, the device layout (face slots, opposite-face pairing,
// boundary-face codes, reflection maps, isothermal table, slab pool), launch
// planning, the per-step launch sequence, the NCCL energy all-reduce and the
// getters.  All arithmetic of the step runs in the kernels of bte_kernels.cuh;
// the host only validates, moves data and plans launches.
#include "../../include/bte.h"
#include "bte_kernels.cuh"
#include "bte_nccl.h"

#include <cudaTypedefs.h>  // PFN_cuTensorMapEncodeTiled (driver entry point, no -lcuda)

#include <algorithm>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <cstdlib>
#include <functional>
#include <array>
#include <map>
#include <mutex>
#include <set>
#include <string>
#include <vector>

namespace {

// CODATA 2018 values (the library's own copy; theta_b = hbar omega_b / kB).
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
enum Phase { kPhFlux = 0, kPhAllreduce = 2, kPhNewton = 3, kPhHalo = 4 };

// One halo segment of a cell-partitioned run: the values this
// rank sends to / receives from one neighbour part, buffers [k][j][i].
struct HaloSeg {
    int part = 0;
    int32_t n_send_cells = 0, n_send_dirs = 0, n_recv_cells = 0, n_recv_dirs = 0, col0 = 0;
    int32_t *send_cells = nullptr, *send_dirs = nullptr, *recv_dirs = nullptr;  // device
    int32_t *recv_cols = nullptr;  // device: halo column of each received cell (relative to pool_cells)
    double *sbuf = nullptr, *rbuf = nullptr;                                      // device
    int64_t n_send() const { return (int64_t)n_send_cells * n_send_dirs; }  // per band-row
    int64_t n_recv() const { return (int64_t)n_recv_cells * n_recv_dirs; }
};

}  // namespace

struct bte_group {
    bte::group::Group *g = nullptr;
};

struct bte_ctx {
    std::string err = "no error";
    bte_options opt{};
    int dim = 0, nd = 0, nb = 0, b_lo = 0, b_hi = 0, nb_loc = 0, mf = 0, mf_t = 0;
    int32_t nc = 0, ps = 0, n_bcells = 0;
    int device = 0;
    int sm_count = 148;
    double W = 0.0, s_max = 0.0, dt_bound = 0.0;
    // slab pool: nb_loc current slabs + n_spare workspace slabs of nd x ps doubles
    double *pool = nullptr;
    double *pool_cells = nullptr;  // pool + the column of the first owned cell (cell index 0); halo
                                   // layers of a z-slab cell partition sit before / after the owned cells
    int64_t slab_elems = 0;
    int n_spare = 0;
    std::vector<int32_t> cur_slot, spare_slot;
    int32_t *d_cur_slot = nullptr;
    double *i0 = nullptr, *T = nullptr, *E = nullptr, *part = nullptr;
    int n_slots_step = 0;
    double *staging = nullptr;
    int64_t staging_elems = 0;
    // face slots [mf_t][nc]
    int32_t *nbr = nullptr, *nbm = nullptr, *pos = nullptr;
    uint32_t *fcode = nullptr;  // paired: 5-bit face codes per cell
    uint8_t *fcode8 = nullptr;  // generic: 8-bit face codes per face slot
    double *gx = nullptr, *gy = nullptr, *gz = nullptr;
    bool paired = false;     // every cell's faces are exact opposite pairs
    bool uniform_g = false;  // ... and every cell has the same g per pair
    bool tma = false;        // 256-thread blocks: the TMA-staged kernel (paired or generic faces)
    int32_t *hl_off = nullptr, *hl_cell = nullptr;  // generic TMA kernel: per-tile halo lists,
    int32_t *bl_off = nullptr, *bl_col = nullptr, *bl_cls = nullptr;  // ... boundary-face ghost lists
    uint16_t *sidx = nullptr;                        // ... per face slot: shared-memory index of the upwind value
    int32_t hstride = 0;
    double gu[3][3] = {};
    // box path (structured hex grid in lexicographic order, flux_box_kernel)
    bool box = false;
    int32_t bn[3] = {0, 0, 0}, bzside[2] = {0, 0};
    bool bflat = false;  // 2-D box grid (no axis-2 faces; isothermal walls on grid axis 1)
    int32_t bz_t = 0, bz_lo = 0;  // z-slab partition: tensor layers (owned + halo), first owned layer
    double bgeo[3] = {0, 0, 0};
    int n_orb = 0, box_L = 8, box_stages = 6, box_nbb = 5, box_oc = 20, box_ctas_per_sm = 2;
    bool td = false;  // temperature-dependent relaxation times (rate tables)
    std::vector<double> h_ra, h_rb, h_rth, h_vg_all, h_inv_tau_all;  // rate law, constants (global rows)
    double *E2 = nullptr, *T2 = nullptr, *cw_diag = nullptr;  // bte_get_temperature_rule scratch
    // band-sharded step (world > 1 with a communicator): reduce-scatter of E,
    // temperature solve on this rank's chunk of cells, all-gather of T
    bool shard_newton = false;
    int32_t nc_pad = 0, chunk = 0;
    double *Echunk = nullptr, *Tg = nullptr;
    double *d_ra = nullptr, *d_rb = nullptr, *d_rth = nullptr, *d_inv_v = nullptr;
    double *rates = nullptr;  // [2][nb_loc][nc]: 1/tau at the rate temperature / at the current T
    double *Tr = nullptr;     // [nc] rate temperature
    double t_hi = 0.0;        // highest temperature the state can reach (dt bound with the law)
    bte::BoxOrbit *orb = nullptr;
    double4 *dirs_box = nullptr;
    double *side_tab = nullptr;
    int32_t *side_col = nullptr;
    CUtensorMap tm_in{}, tm_out{}, tm_i0{}, tm_side{}, tm_rate{};
    int rsel = 0;  // rate tables: which half holds the current rates
    // boundary faces: reflection maps of specular classes, isothermal table
    int32_t *refl = nullptr;
    int32_t n_iso = 0, n_refl = 0;
    double *i0w = nullptr, *twall = nullptr;
    // tables
    double4 *dirs = nullptr;
    double *cw_loc = nullptr;
    std::vector<double> h_inv_tau, h_vg, h_cw;  // local band-rows
    double *Cb = nullptr, *theta = nullptr, *cw_all = nullptr;
    int32_t *d_iter_max = nullptr;
    // d_flags[0] fail (a temperature solve failed), [1] halt (the fail flag as the
    // step's flux launch saw it: the rest of the step is a no-op), [2] steps done
    // (counted by each step's last kernel; the host undoes the slab rotation of
    // the steps skipped after a failure, so the state is that of the failing step)
    int32_t *d_flags = nullptr, *d_fail = nullptr, *d_halt = nullptr, *d_done = nullptr;
    int32_t done_seen = 0;
    int newton_mode = 0;  // the step's solve: 0 by mesh size, 1 warp per cell, 2 thread per cell
    unsigned long long *d_smax = nullptr;
    // launch plan
    int bg = 4, block = 256;
    int dir_chunks = 1;
    // execution
    cudaStream_t stream = nullptr;
    bool own_stream = false;
    bte::nccl::Comm comm{};
    bool have_comm = false;
    // cell partitioning (N3): part of this rank, band groups, halo segments;
    // the energy is reduced over the ranks of the same part (bcomm, G ranks)
    int n_parts = 1, my_part = 0, G = 1, gband = 0;
    int32_t n_halo = 0;
    std::vector<HaloSeg> hsegs;
    std::vector<int64_t> gid;  // owned cells: global ids ascending (caller order of the ABI)
    bte::nccl::Comm bcomm{};
    bool have_bcomm = false, own_bcomm = false;
    bool begun = false;  // split step in flight
    // CUDA graph of two steps (double-buffered single-GPU runs: after two steps the
    // slab pointers and rate halves are back where they were, so it replays)
    cudaGraphExec_t gexec = nullptr;
    double g_dt = 0.0;
    int g_key = -1;
    int64_t g_launches = 0, g_flux = 0;
    bool graphs_ok = true;
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
// Dynamic shared memory above 48 KB needs a per-function opt-in, and the
// attribute belongs to the device's context: remembered per (device, function),
// raised only (contexts with different layouts need different amounts).
cudaError_t ensure_smem(const void *fn, size_t smem) {
    if (smem <= 48 * 1024) return cudaSuccess;
    static std::mutex mu;
    static std::map<std::pair<int, const void *>, size_t> granted;
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return e;
    std::lock_guard<std::mutex> lk(mu);
    size_t &g = granted[{dev, fn}];
    if (smem <= g) return cudaSuccess;
    e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e == cudaSuccess) g = smem;
    return e;
}

using FluxLaunch = cudaError_t (*)(dim3, dim3, cudaStream_t, const bte::FluxParams &);

// Register-pipelined generic-face kernel (block sizes other than 256, or meshes
// whose tiles stage too many halo / ghost values for the TMA kernel).
template <int DIM, int MF, int BG>
cudaError_t flux_launch_t(dim3 g, dim3 b, cudaStream_t s, const bte::FluxParams &p) {
    bte::flux_kernel<DIM, MF, BG><<<g, b, 0, s>>>(p);
    return cudaGetLastError();
}

// TMA-staged paired kernel: one 256-cell tile per block, kStages x BG x 2 KB ring.
template <int DIM, int NP, int BG, bool UG>
cudaError_t flux_tma_launch_t(dim3 g, dim3, cudaStream_t s, const bte::FluxParams &p) {
    const size_t smem = (size_t)bte::kStages * BG * bte::kTile * sizeof(double) +
                        (UG ? (size_t)p.dchunk * sizeof(bte::DirEntry<NP>) : 0);
    cudaError_t e = ensure_smem((const void *)bte::flux_tma_kernel<DIM, NP, BG, UG>, smem);
    if (e != cudaSuccess) return e;
    bte::flux_tma_kernel<DIM, NP, BG, UG><<<g, dim3(bte::kTmaThreads), smem, s>>>(p);
    return cudaGetLastError();
}

// TMA-staged generic-face kernel (general meshes): kStages x BG x 2 KB ring.
template <int DIM, int MF, int BG, bool TD>
cudaError_t flux_tma_generic_launch_td(dim3 g, const bte::FluxParams &p, cudaStream_t s) {
    const size_t smem = (size_t)bte::kStagesG * BG * p.hstride * sizeof(double) + (size_t)p.dchunk * sizeof(double4);
    cudaError_t e = ensure_smem((const void *)bte::flux_tma_generic_kernel<DIM, MF, BG, TD>, smem);
    if (e != cudaSuccess) return e;
    bte::flux_tma_generic_kernel<DIM, MF, BG, TD><<<g, dim3(bte::kTmaThreads), smem, s>>>(p);
    return cudaGetLastError();
}

template <int DIM, int MF, int BG>
cudaError_t flux_tma_generic_launch_t(dim3 g, dim3, cudaStream_t s, const bte::FluxParams &p) {
    if (p.rate_cur) return flux_tma_generic_launch_td<DIM, MF, BG, true>(g, p, s);
    return flux_tma_generic_launch_td<DIM, MF, BG, false>(g, p, s);
}

template <int DIM, int MF>
FluxLaunch pick_tma_generic(int bg) {
    switch (bg) {
        case 1: return flux_tma_generic_launch_t<DIM, MF, 1>;
        case 2: return flux_tma_generic_launch_t<DIM, MF, 2>;
        default: return flux_tma_generic_launch_t<DIM, MF, 4>;
    }
}

template <int DIM, int NP, bool UG>
FluxLaunch pick_tma(int bg) {
    switch (bg) {
        case 1: return flux_tma_launch_t<DIM, NP, 1, UG>;
        case 2: return flux_tma_launch_t<DIM, NP, 2, UG>;
        case 3: return flux_tma_launch_t<DIM, NP, 3, UG>;
        case 4: return flux_tma_launch_t<DIM, NP, 4, UG>;
        case 5: return flux_tma_launch_t<DIM, NP, 5, UG>;
        case 6: return flux_tma_launch_t<DIM, NP, 6, UG>;
        case 7: return flux_tma_launch_t<DIM, NP, 7, UG>;
        default: return flux_tma_launch_t<DIM, NP, 8, UG>;
    }
}

// Generic register kernels exist for band groups 1, 2, 4.
template <int DIM, int MF>
FluxLaunch pick_generic(int bg) {
    switch (bg) {
        case 1: return flux_launch_t<DIM, MF, 1>;
        case 2: return flux_launch_t<DIM, MF, 2>;
        default: return flux_launch_t<DIM, MF, 4>;
    }
}

// mf_t: padded faces per cell (generic) or face pairs per cell (paired; paired
// layouts are only built for the TMA kernel)
FluxLaunch pick_flux(int dim, int mf_t, int bg, bool paired, bool uniform_g, bool tma) {
    if (paired) {
        if (uniform_g) return dim == 2 ? pick_tma<2, 2, true>(bg) : pick_tma<3, 3, true>(bg);
        return dim == 2 ? pick_tma<2, 2, false>(bg) : pick_tma<3, 3, false>(bg);
    }
    if (tma) {
        if (dim == 2) return mf_t == 3 ? pick_tma_generic<2, 3>(bg) : mf_t == 4 ? pick_tma_generic<2, 4>(bg)
                                                                               : pick_tma_generic<2, 8>(bg);
        return mf_t == 4 ? pick_tma_generic<3, 4>(bg) : mf_t == 6 ? pick_tma_generic<3, 6>(bg)
                                                                  : pick_tma_generic<3, 8>(bg);
    }
    if (dim == 2) return mf_t == 3 ? pick_generic<2, 3>(bg) : mf_t == 4 ? pick_generic<2, 4>(bg) : pick_generic<2, 8>(bg);
    return mf_t == 4 ? pick_generic<3, 4>(bg) : mf_t == 6 ? pick_generic<3, 6>(bg) : pick_generic<3, 8>(bg);
}

int legal_bg(int bg, bool paired) {
    bg = std::max(1, std::min(8, bg));
    if (paired) return bg;
    return bg <= 1 ? 1 : bg <= 3 ? 2 : 4;
}

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

// ------------------------------------------------------------- box path
// Structured hexahedral grid detection (flux_box_kernel): every cell has six
// faces with normals exactly +-e_a, the face graph is an n_0 x n_1 x n_2
// lattice (walked from the corner cell), A_f / V_c is the same for every cell
// per axis, and each of the six sides is uniformly isothermal or specular with
// isothermal faces on at most one axis.  That axis (else mesh z) becomes grid
// axis 2 (the marching axis); grid axis 0 (contiguous) is a remaining axis of
// even extent (16-byte tensor strides).  cell_at lists the user cells in grid
// lexicographic order.
struct BoxDetect {
    bool ok = false;
    int ax[3] = {0, 1, 2};      // grid axis -> mesh axis
    int32_t n[3] = {0, 0, 0};   // extents along grid axes
    double g[3] = {0, 0, 0};    // A / V along grid axes
    int zside[2] = {1, 1};      // ghost axis (3-D: grid axis 2; 2-D: grid axis 1) low / high side:
                                // 0 isothermal, 1 specular
    bool flat = false;          // 2-D grid: n[2] = 1, no axis-2 faces (g[2] = 0)
    std::vector<int32_t> cell_at;
    std::vector<int64_t> zbface[2];  // boundary face ids of the ghost-axis sides: 3-D [n1][n0], 2-D [n0]
};

// 2-D structured quad grid (the paper's Fig.-1 and Fig.-10 meshes): four faces
// per cell with normals exactly +-e_x, +-e_y, an n_0 x n_1 lattice, uniform
// A / V per axis, each side uniformly isothermal or specular with isothermal
// sides on at most one axis, which becomes grid axis 1 (its wall ghosts are
// staged rows of I0_b(T_wall), Eq. 6); grid axis 0 (contiguous, specular
// sides) must have even extent.  Grid axis 2 is a single layer with no faces.
BoxDetect detect_box2d(const bte_mesh *m, const bte_bcs *bc) {
    BoxDetect r;
    if (m->dim != 2) return r;
    const int64_t nc = m->n_cells;
    std::vector<int64_t> fa((size_t)nc * 4, -1);  // [cell][2 axis + (normal > 0)] -> face
    for (int64_t c = 0; c < nc; ++c) {
        if (m->face_offsets[c + 1] - m->face_offsets[c] != 4) return r;
        for (int64_t f = m->face_offsets[c]; f < m->face_offsets[c + 1]; ++f) {
            const double *nv = m->face_normal + 3 * f;
            int a = -1;
            for (int t = 0; t < 2; ++t)
                if (nv[t] == 1.0 || nv[t] == -1.0) a = t;
            if (a < 0 || nv[1 - a] != 0.0 || nv[2] != 0.0) return r;
            int64_t &slot = fa[(size_t)c * 4 + 2 * a + (nv[a] > 0.0)];
            if (slot >= 0) return r;
            slot = f;
        }
    }
    auto nbr = [&](int64_t c, int a, int sd) { return m->face_nbr[fa[(size_t)c * 4 + 2 * a + sd]]; };
    int64_t corner = -1;
    for (int64_t c = 0; c < nc && corner < 0; ++c)
        if (nbr(c, 0, 0) < 0 && nbr(c, 1, 0) < 0) corner = c;
    if (corner < 0) return r;
    int64_t n[2];
    for (int a = 0; a < 2; ++a) {
        n[a] = 1;
        for (int64_t c = corner; nbr(c, a, 1) >= 0; c = nbr(c, a, 1))
            if (++n[a] > nc) return r;
    }
    if (n[0] * n[1] != nc) return r;
    std::vector<int32_t> at(nc, -1);  // mesh-axis lexicographic position -> cell
    std::vector<char> seen(nc, 0);
    int64_t ys = corner;
    for (int64_t y = 0; y < n[1]; ++y) {
        if (y > 0 && (ys = nbr(ys, 1, 1)) < 0) return r;
        int64_t c = ys;
        for (int64_t x = 0; x < n[0]; ++x) {
            if (x > 0 && (c = nbr(c, 0, 1)) < 0) return r;
            if (seen[c]) return r;
            seen[c] = 1;
            at[y * n[0] + x] = (int32_t)c;
        }
    }
    int kind[2][2] = {{-1, -1}, {-1, -1}};  // -1 none yet, 0 iso, 1 sym, 2 mixed
    double g[2];
    for (int a = 0; a < 2; ++a) g[a] = m->face_area[fa[(size_t)at[0] * 4 + 2 * a + 1]] / m->cell_volume[at[0]];
    for (int64_t y = 0; y < n[1]; ++y)
        for (int64_t x = 0; x < n[0]; ++x) {
            const int64_t p[2] = {x, y};
            const int64_t c = at[y * n[0] + x];
            for (int a = 0; a < 2; ++a)
                for (int sd = 0; sd < 2; ++sd) {
                    const int64_t f = fa[(size_t)c * 4 + 2 * a + sd];
                    if (m->face_area[f] / m->cell_volume[c] != g[a]) return r;
                    int64_t q[2] = {p[0], p[1]};
                    q[a] += sd ? 1 : -1;
                    const int64_t v = m->face_nbr[f];
                    if (q[a] >= 0 && q[a] < n[a]) {
                        if (v != at[q[1] * n[0] + q[0]]) return r;
                    } else {
                        if (v >= 0) return r;
                        const int k = bc->kind[-1 - v] == BTE_BC_ISOTHERMAL ? 0 : 1;
                        int &s = kind[a][sd];
                        s = s < 0 ? k : (s == k ? k : 2);
                    }
                }
        }
    int isoax = -1;
    for (int a = 0; a < 2; ++a) {
        if (kind[a][0] == 2 || kind[a][1] == 2) return r;
        if (kind[a][0] == 0 || kind[a][1] == 0) {
            if (isoax >= 0) return r;
            isoax = a;
        }
    }
    if (isoax >= 0) r.ax[0] = 1 - isoax, r.ax[1] = isoax;
    else if (n[0] % 2 == 0) r.ax[0] = 0, r.ax[1] = 1;
    else r.ax[0] = 1, r.ax[1] = 0;
    r.ax[2] = 2;
    if (n[r.ax[0]] % 2 != 0) return r;
    r.flat = true;
    for (int t = 0; t < 2; ++t) r.n[t] = (int32_t)n[r.ax[t]], r.g[t] = g[r.ax[t]];
    r.n[2] = 1;
    r.g[2] = 0.0;
    for (int sd = 0; sd < 2; ++sd) r.zside[sd] = kind[r.ax[1]][sd];
    r.cell_at.resize(nc);
    for (int sd = 0; sd < 2; ++sd) r.zbface[sd].assign((size_t)r.n[0], -1);
    for (int64_t i1 = 0; i1 < r.n[1]; ++i1)
        for (int64_t i0 = 0; i0 < r.n[0]; ++i0) {
            int64_t p[2];
            p[r.ax[0]] = i0, p[r.ax[1]] = i1;
            const int32_t c = at[p[1] * n[0] + p[0]];
            r.cell_at[i1 * r.n[0] + i0] = c;
            for (int sd = 0; sd < 2; ++sd)
                if (i1 == (sd ? r.n[1] - 1 : 0)) r.zbface[sd][i0] = -1 - nbr(c, r.ax[1], sd);
        }
    r.ok = true;
    return r;
}

BoxDetect detect_box(const bte_mesh *m, const bte_bcs *bc) {
    BoxDetect r;
    if (m->dim != 3) return r;
    const int64_t nc = m->n_cells;
    std::vector<int64_t> fa((size_t)nc * 6, -1);  // [cell][2 axis + (normal > 0)] -> face
    for (int64_t c = 0; c < nc; ++c) {
        if (m->face_offsets[c + 1] - m->face_offsets[c] != 6) return r;
        for (int64_t f = m->face_offsets[c]; f < m->face_offsets[c + 1]; ++f) {
            const double *nv = m->face_normal + 3 * f;
            int a = -1;
            for (int t = 0; t < 3; ++t)
                if (nv[t] == 1.0 || nv[t] == -1.0) a = t;
            if (a < 0 || nv[(a + 1) % 3] != 0.0 || nv[(a + 2) % 3] != 0.0) return r;
            int64_t &slot = fa[(size_t)c * 6 + 2 * a + (nv[a] > 0.0)];
            if (slot >= 0) return r;
            slot = f;
        }
    }
    auto nbr = [&](int64_t c, int a, int sd) { return m->face_nbr[fa[(size_t)c * 6 + 2 * a + sd]]; };
    int64_t corner = -1;
    for (int64_t c = 0; c < nc && corner < 0; ++c)
        if (nbr(c, 0, 0) < 0 && nbr(c, 1, 0) < 0 && nbr(c, 2, 0) < 0) corner = c;
    if (corner < 0) return r;
    int64_t n[3];
    for (int a = 0; a < 3; ++a) {
        n[a] = 1;
        for (int64_t c = corner; nbr(c, a, 1) >= 0; c = nbr(c, a, 1))
            if (++n[a] > nc) return r;
    }
    if (n[0] * n[1] * n[2] != nc) return r;
    std::vector<int32_t> at(nc, -1);  // mesh-axis lexicographic position -> cell
    std::vector<char> seen(nc, 0);
    int64_t zs = corner;
    for (int64_t z = 0; z < n[2]; ++z) {
        if (z > 0 && (zs = nbr(zs, 2, 1)) < 0) return r;
        int64_t ys = zs;
        for (int64_t y = 0; y < n[1]; ++y) {
            if (y > 0 && (ys = nbr(ys, 1, 1)) < 0) return r;
            int64_t c = ys;
            for (int64_t x = 0; x < n[0]; ++x) {
                if (x > 0 && (c = nbr(c, 0, 1)) < 0) return r;
                if (seen[c]) return r;
                seen[c] = 1;
                at[(z * n[1] + y) * n[0] + x] = (int32_t)c;
            }
        }
    }
    int kind[3][2] = {{-1, -1}, {-1, -1}, {-1, -1}};  // -1 none yet, 0 iso, 1 sym, 2 mixed
    double g[3];
    for (int a = 0; a < 3; ++a) g[a] = m->face_area[fa[(size_t)at[0] * 6 + 2 * a + 1]] / m->cell_volume[at[0]];
    for (int64_t z = 0; z < n[2]; ++z)
        for (int64_t y = 0; y < n[1]; ++y)
            for (int64_t x = 0; x < n[0]; ++x) {
                const int64_t p[3] = {x, y, z};
                const int64_t c = at[(z * n[1] + y) * n[0] + x];
                for (int a = 0; a < 3; ++a)
                    for (int sd = 0; sd < 2; ++sd) {
                        const int64_t f = fa[(size_t)c * 6 + 2 * a + sd];
                        if (m->face_area[f] / m->cell_volume[c] != g[a]) return r;
                        int64_t q[3] = {p[0], p[1], p[2]};
                        q[a] += sd ? 1 : -1;
                        const int64_t v = m->face_nbr[f];
                        if (q[a] >= 0 && q[a] < n[a]) {
                            if (v != at[(q[2] * n[1] + q[1]) * n[0] + q[0]]) return r;
                        } else {
                            if (v >= 0) return r;
                            const int k = bc->kind[-1 - v] == BTE_BC_ISOTHERMAL ? 0 : 1;
                            int &s = kind[a][sd];
                            s = s < 0 ? k : (s == k ? k : 2);
                        }
                    }
            }
    int isoax = -1;
    for (int a = 0; a < 3; ++a) {
        if (kind[a][0] == 2 || kind[a][1] == 2) return r;
        if (kind[a][0] == 0 || kind[a][1] == 0) {
            if (isoax >= 0) return r;
            isoax = a;
        }
    }
    r.ax[2] = isoax >= 0 ? isoax : 2;
    int rest[2], nr = 0;
    for (int a = 0; a < 3; ++a)
        if (a != r.ax[2]) rest[nr++] = a;
    if (n[rest[0]] % 2 == 0) r.ax[0] = rest[0], r.ax[1] = rest[1];
    else if (n[rest[1]] % 2 == 0) r.ax[0] = rest[1], r.ax[1] = rest[0];
    else return r;
    for (int t = 0; t < 3; ++t) r.n[t] = (int32_t)n[r.ax[t]], r.g[t] = g[r.ax[t]];
    for (int sd = 0; sd < 2; ++sd) r.zside[sd] = kind[r.ax[2]][sd];
    r.cell_at.resize(nc);
    for (int sd = 0; sd < 2; ++sd) r.zbface[sd].assign((size_t)r.n[0] * r.n[1], -1);
    for (int64_t i2 = 0; i2 < r.n[2]; ++i2)
        for (int64_t i1 = 0; i1 < r.n[1]; ++i1)
            for (int64_t i0 = 0; i0 < r.n[0]; ++i0) {
                int64_t p[3];
                p[r.ax[0]] = i0, p[r.ax[1]] = i1, p[r.ax[2]] = i2;
                const int32_t c = at[(p[2] * n[1] + p[1]) * n[0] + p[0]];
                r.cell_at[(i2 * r.n[1] + i1) * r.n[0] + i0] = c;
                for (int sd = 0; sd < 2; ++sd)
                    if (i2 == (sd ? r.n[2] - 1 : 0))
                        r.zbface[sd][i1 * r.n[0] + i0] = -1 - nbr(c, r.ax[2], sd);
            }
    r.ok = true;
    return r;
}

// Orbits of the direction set under the grid axis-0 and axis-1 mirrors (both
// pairs of sides are specular, so the set is closed under them; Eq. 6).  Every
// orbit must have four members (no direction with s_0 = 0 or s_1 = 0).  rz:
// axis-2 mirror, needed when an axis-2 side is specular.
bool box_orbits(const bte_dirs *dr, const int ax[3], bool need_rz, std::vector<bte::BoxOrbit> *out) {
    const int nd = dr->n_dirs;
    auto mirror = [&](int d, int a) {
        const double *s = dr->s + 3 * d;
        double r[3] = {s[0], s[1], s[2]};
        r[a] = -r[a];
        for (int e = 0; e < nd; ++e) {
            const double *t = dr->s + 3 * e;
            if (std::fabs(t[0] - r[0]) <= 1e-10 && std::fabs(t[1] - r[1]) <= 1e-10 && std::fabs(t[2] - r[2]) <= 1e-10)
                return e;
        }
        return -1;
    };
    std::vector<int> m0(nd), m1(nd), m2(nd, -1);
    for (int d = 0; d < nd; ++d) {
        if (dr->s[3 * d + ax[0]] == 0.0 || dr->s[3 * d + ax[1]] == 0.0) return false;
        m0[d] = mirror(d, ax[0]);
        m1[d] = mirror(d, ax[1]);
        if (need_rz) m2[d] = mirror(d, ax[2]);
        if (m0[d] < 0 || m1[d] < 0 || (need_rz && m2[d] < 0)) return false;
    }
    std::vector<char> used(nd, 0);
    out->clear();
    for (int d = 0; d < nd; ++d) {
        if (used[d]) continue;
        int b = dr->s[3 * d + ax[0]] > 0.0 ? d : m0[d];
        b = dr->s[3 * b + ax[1]] > 0.0 ? b : m1[b];
        const int q[4] = {b, m0[b], m1[b], m0[m1[b]]};
        if (m1[m0[b]] != q[3]) return false;
        bte::BoxOrbit o;
        for (int j = 0; j < 4; ++j) {
            if (used[q[j]]) return false;
            used[q[j]] = 1;
            o.d[j] = q[j];
            o.rz[j] = need_rz ? m2[q[j]] : -1;
        }
        out->push_back(o);
    }
    return true;
}

PFN_cuTensorMapEncodeTiled_v12000 tensor_map_encoder() {
    static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
    if (!fn) {
        void *p = nullptr;
        cudaDriverEntryPointQueryResult q{};
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
    }
    return fn;
}

// FP64 tiled tensor map; dims/box innermost first, strides in bytes for dims 1..rank-1.
bool encode_map(CUtensorMap *tm, void *base, int rank, const uint64_t *dims, const uint64_t *strides,
                const uint32_t *box) {
    auto fn = tensor_map_encoder();
    if (!fn) return false;
    cuuint64_t gd[5], gs[4];
    cuuint32_t bx[5], es[5];
    for (int i = 0; i < rank; ++i) gd[i] = dims[i], bx[i] = box[i], es[i] = 1;
    for (int i = 0; i + 1 < rank; ++i) gs[i] = strides[i];
    return fn(tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, (cuuint32_t)rank, base, gd, gs, bx, es,
              CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
              CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

// Launch geometry of the box kernel.  Work item = one 32 x 8 x L cell block x
// nbb band-rows x oc orbits; persistent CTAs (sm_count x resident CTAs per
// SM) take the items round-robin, tile fastest.  Defaults (measured on B200,
// DESIGN.md 10): nbb = 5 band-rows, oc = the largest divisor of n_orb <= 20
// (whole chunks: a ragged last chunk idles part of the grid); the options
// band_group / dir_chunk override them.  One energy slot per (band batch,
// orbit chunk).
struct BoxPlan {
    int tiles0, tiles1, zranges, n_batches, n_chunks, nbb, oc;
};
constexpr int kBoxMaxOrbChunk = 32;  // orbits per item (shared-memory orbit table)

BoxPlan plan_box(const bte_ctx *ctx, int nbl) {
    BoxPlan b;
    b.tiles0 = (ctx->bn[0] + bte::kBoxTX - 1) / bte::kBoxTX;
    b.tiles1 = (ctx->bn[1] + bte::kBoxTY - 1) / bte::kBoxTY;
    b.zranges = (ctx->bn[2] + ctx->box_L - 1) / ctx->box_L;
    // band-rows per item (measured on B200): up to 5 when a
    // slice's tiles all fit in the resident CTAs (C4), the largest that still
    // gives >= 8 waves of CTAs (band-sharded launches have few rows); 1 when a
    // slice has more tiles than resident CTAs, so it is swept quickly and
    // neighbouring tiles stay close in time (C5)
    const int tiles = b.tiles0 * b.tiles1 * b.zranges;
    const int64_t slots = (int64_t)ctx->sm_count * ctx->box_ctas_per_sm;
    int oc_pre = 1;
    for (int c = std::min({ctx->n_orb, kBoxMaxOrbChunk, ctx->box_oc}); c >= 1; --c)
        if (ctx->n_orb % c == 0) {
            oc_pre = c;
            break;
        }
    if (ctx->opt.dir_chunk > 0) oc_pre = std::max(1, std::min({ctx->n_orb, kBoxMaxOrbChunk, (int)ctx->opt.dir_chunk / 4}));
    int auto_nbb = 1;
    if (tiles <= slots)
        for (int n = std::min(nbl, ctx->box_nbb); n >= 1; --n) {
            const int64_t ctas = (int64_t)tiles * ((nbl + n - 1) / n) * ((ctx->n_orb + oc_pre - 1) / oc_pre);
            if (ctas >= 8 * slots) {
                auto_nbb = n;
                break;
            }
        }
    b.nbb = std::min(nbl, ctx->opt.band_group > 0 ? (int)ctx->opt.band_group : auto_nbb);
    if (ctx->opt.dir_chunk > 0) {
        b.oc = std::max(1, std::min({ctx->n_orb, kBoxMaxOrbChunk, (int)ctx->opt.dir_chunk / 4}));
    } else {
        b.oc = oc_pre;
        // 3-D launches whose items got one row each (few band-rows per launch: band
        // sharding over 4-8 GPUs): the most rows per item, then the largest orbit
        // chunk, that still give 8 waves (measured on B200, C4 emulated ranks: 7 rows
        // 0.994 -> 0.958 ms with 5 rows x 5 orbits instead of 1 x 20; 14 rows 1.942 ->
        // 1.879 ms)
        if (!ctx->bflat && tiles <= slots && auto_nbb == 1 && ctx->opt.band_group <= 0) {
            bool done = false;
            for (int n = std::min(nbl, ctx->box_nbb); n >= 1 && !done; --n)
                for (int c = oc_pre; c >= 1 && !done; --c) {
                    if (ctx->n_orb % c) continue;
                    if ((int64_t)tiles * ((nbl + n - 1) / n) * (ctx->n_orb / c) >= 8 * slots) {
                        b.oc = c;
                        b.nbb = n;
                        done = true;
                    }
                }
        }
    }
    b.n_batches = (nbl + b.nbb - 1) / b.nbb;
    b.n_chunks = (ctx->n_orb + b.oc - 1) / b.oc;
    return b;
}

// doubles per ring stage (2-D: + the two isothermal wall rows of grid axis 1)
int box_stage(const bte_ctx *ctx) {
    return (ctx->td ? bte::box_stage_elems<true>() : bte::box_stage_elems<false>()) + (ctx->bflat ? 2 * bte::kBoxTX : 0);
}

size_t box_smem(const bte_ctx *ctx) {
    const int stage = box_stage(ctx);
#ifdef BTE_BOX_TMA_STORE
    constexpr size_t obuf = 2 * 4 * bte::kBoxCells;  // double-buffered output tiles of the tensor stores
#else
    constexpr size_t obuf = 0;  // results leave straight from registers
#endif
    return ((size_t)ctx->box_stages * stage + obuf + (size_t)ctx->box_L * bte::kBoxCells) *
               sizeof(double) +
           (size_t)kBoxMaxOrbChunk * sizeof(bte::BoxOrbitC);
}

// The box kernel instantiation of a context: rate tables or not, 2-D (3 CTAs
// per SM) or 3-D (2).
using BoxKernel = void (*)(const bte::BoxParams, const CUtensorMap, const CUtensorMap, const CUtensorMap,
                           const CUtensorMap, const CUtensorMap);
BoxKernel box_kernel(const bte_ctx *ctx) {
    if (ctx->bflat) return ctx->td ? bte::flux_box_kernel<true, true> : bte::flux_box_kernel<false, true>;
    return ctx->td ? bte::flux_box_kernel<true, false> : bte::flux_box_kernel<false, false>;
}

bte_status box_setup_kernel(bte_ctx *ctx) {
    const size_t smem = box_smem(ctx);
    // the attribute is per function, shared by every context of the process: only ever raise it
    // (contexts with different layer ranges need different amounts)
    static std::map<const void *, size_t> granted;
    size_t &g = granted[(const void *)box_kernel(ctx)];
    if (smem > g) {
        CUDA_TRY(ctx, cudaFuncSetAttribute(box_kernel(ctx), cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
        g = smem;
    }
    int occ = 0;
    CUDA_TRY(ctx, cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, box_kernel(ctx), bte::kBoxThreads, smem));
    ctx->box_ctas_per_sm = std::max(1, occ);
    return BTE_OK;
}

// Rate tables (N1): half `sel` of ctx->rates.
double *rate_half(bte_ctx *ctx, int sel) { return ctx->rates + (size_t)sel * ctx->nb_loc * ctx->nc; }

// ------------------------------------------------------------- launch plan
struct LaunchPlan {
    int groups, n_dch, dchunk;
};

// A band batch of nbl rows is launched as segments of full band groups: the
// largest multiple of bg first, then the remainder as one smaller group
// (paired kernels: any size 1..8) or as power-of-two groups (generic kernels).
struct Segment {
    int off, nbl, bg;
};
std::vector<Segment> segments(int nbl, int bg, bool paired) {
    std::vector<Segment> out;
    int off = 0;
    while (off < nbl) {
        int g = std::min(bg, nbl - off);
        if (!paired)
            while (g & (g - 1)) g &= g - 1;  // largest power of two <= g
        const int n = (nbl - off) / g * g;
        out.push_back({off, n, g});
        off += n;
    }
    return out;
}

// Direction chunks: at most kAutoDirChunk directions per block (short blocks
// keep the tiles that share halo data resident at the same time, so upwind
// reads hit L2; measured best on B200) and enough chunks for the
// grid to hold ~2 full waves of threads.
constexpr int kAutoDirChunk = 40;
LaunchPlan plan_launch(const bte_ctx *ctx, int nbl, int bg) {
    LaunchPlan lp;
    lp.groups = nbl / bg;
    const int64_t target = (int64_t)ctx->sm_count * 2048 * 2;
    const int64_t have = std::max<int64_t>(1, (int64_t)ctx->nc * lp.groups);
    const int n = (int)std::min<int64_t>(ctx->nd, std::max<int64_t>(1, (target + have - 1) / have));
    lp.dchunk = (ctx->nd + n - 1) / n;
    lp.dchunk = std::min(lp.dchunk, ctx->opt.dir_chunk > 0 ? (int)ctx->opt.dir_chunk : kAutoDirChunk);
    lp.n_dch = (ctx->nd + lp.dchunk - 1) / lp.dchunk;
    return lp;
}

int count_slots(const bte_ctx *ctx) {
    int slots = 0;
    if (ctx->box) {
        for (int l0 = 0; l0 < ctx->nb_loc; l0 += ctx->n_spare) {
            const BoxPlan bp = plan_box(ctx, std::min(ctx->n_spare, ctx->nb_loc - l0));
            slots += bp.n_batches * bp.n_chunks;
        }
        return slots;
    }
    for (int l0 = 0; l0 < ctx->nb_loc; l0 += ctx->n_spare)
        for (const Segment &sg : segments(std::min(ctx->n_spare, ctx->nb_loc - l0), ctx->bg, ctx->paired)) {
            const LaunchPlan lp = plan_launch(ctx, sg.nbl, sg.bg);
            slots += lp.groups * lp.n_dch;
        }
    return slots;
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
    p.rsel_next = 1 - ctx->rsel;
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
    p.bl_off = ctx->bl_off;
    p.bl_col = ctx->bl_col;
    p.bl_cls = ctx->bl_cls;
    p.sidx = ctx->sidx;
    p.hstride = ctx->hstride;
    p.fail = ctx->d_fail;
    p.halt = ctx->d_halt;
    if (ctx->td) {
        p.rate_cur = rate_half(ctx, ctx->rsel);
        p.rate_next = rate_half(ctx, 1 - ctx->rsel);
        p.rate_r2 = ctx->opt.temp_rule == 0;
    }
    int slot = 0;
    const dim3 block(ctx->block);
    for (int l0 = 0; l0 < ctx->nb_loc; l0 += ctx->n_spare) {
        const int nbl_batch = std::min(ctx->n_spare, ctx->nb_loc - l0);
        for (const Segment &sg : segments(nbl_batch, ctx->bg, ctx->paired)) {
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

// step: the solve that ends a step (rate temperature <- T^n, weights at T^n,
// the new rates go to the current half, which the caller then swaps); else a
// re-solve of the current state (weights at the kept rate temperature, the
// new rates go to the "next" half).
bte::NewtonParams newton_params(bte_ctx *ctx, const double *E_or_null, bool step);

bte_status newton_finish(bte_ctx *ctx);
bte_status reduce_slots(bte_ctx *ctx);

// The step's temperature solve.  Small meshes (fewer cells than ~8 warps of
// threads per SM): E (the slot sum unless reduced already) -> one warp per cell
// (newton_warp_kernel) -> the epilogue (T, Tr, I0, rates); measured on B200,
// C3 (14,400 cells) 0.066 -> 0.053 ms.  Larger meshes: one thread per cell
// (newton_kernel, one launch; C4 0.16 ms vs 0.21 with warps).  Re-solves of the
// current state (step = false) use newton_kernel.
bool warp_newton(const bte_ctx *ctx, int ncells) {
    if (ctx->newton_mode) return ctx->newton_mode == 1;  // (BTE_NEWTON=warp|thread: tests of both kernels)
    return ncells < 32 * 8 * ctx->sm_count;
}

// Band constants in shared memory: C, theta, c_b (+ the four rate-law arrays).
size_t newton_smem(const bte_ctx *ctx) { return (size_t)(ctx->td ? 7 : 3) * ctx->nb * sizeof(double); }

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

// Warp-per-cell solve: R = band-rows per lane, the smallest power of two >= nb / 32.
template <int R>
bte_status launch_newton_warp_r(bte_ctx *ctx, const bte::NewtonParams &q) {
    CUDA_TRY(ctx, ensure_smem((const void *)bte::newton_warp_kernel<R>, newton_smem(ctx)));
    bte::newton_warp_kernel<R><<<(q.nc + 7) / 8, 256, newton_smem(ctx), ctx->stream>>>(q);
    ctx->st.kernel_launches++;
    CUDA_TRY(ctx, cudaGetLastError());
    return BTE_OK;
}

bte_status launch_newton_warp(bte_ctx *ctx, const bte::NewtonParams &q) {
    if (q.nc <= 0) return BTE_OK;
    const int r = (ctx->nb + 31) / 32;
    if (r <= 2) return launch_newton_warp_r<2>(ctx, q);
    if (r <= 4) return launch_newton_warp_r<4>(ctx, q);
    if (r <= 8) return launch_newton_warp_r<8>(ctx, q);
    if (r <= 16) return launch_newton_warp_r<16>(ctx, q);
    static_assert(bte::kMaxBands <= 32 * 32, "warp solve: at most 32 band-rows per lane");
    return launch_newton_warp_r<32>(ctx, q);
}

bte_status run_newton(bte_ctx *ctx, const double *E_or_null, bool step = true) {
    if (step && warp_newton(ctx, ctx->nc)) {
        ev_mark(ctx, kPhNewton, true);
        if (!E_or_null) {
            STATUS_TRY(reduce_slots(ctx));
            E_or_null = ctx->E;
        }
        bte::NewtonParams q = newton_params(ctx, E_or_null, true);
        q.T_out = ctx->Tg;
        q.neg_fail = 1;
        STATUS_TRY(launch_newton_warp(ctx, q));
        STATUS_TRY(newton_finish(ctx));
        ev_mark(ctx, kPhNewton, false);
        if (ctx->td) ctx->rsel = 1 - ctx->rsel;
        return BTE_OK;
    }
    bte::NewtonParams q = newton_params(ctx, E_or_null, step);
    if (step) q.done = ctx->d_done;  // the step's last kernel
    ev_mark(ctx, kPhNewton, true);
    STATUS_TRY(launch_newton_cells(ctx, q));
    ev_mark(ctx, kPhNewton, false);
    if (ctx->td && step) ctx->rsel = 1 - ctx->rsel;
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
        q.rate_out = rate_half(ctx, step ? ctx->rsel : 1 - ctx->rsel);
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
    q.maxit = ctx->opt.newton_max_iter;
    q.iter_max = ctx->d_iter_max;
    q.fail = ctx->d_fail;
    q.single = ctx->opt.temp_rule == 2;
    if (step) q.halt = ctx->d_halt;  // (a step's solve: no-op after a failure earlier in the call)
    return q;
}

bte_status allreduce_E(bte_ctx *ctx, double *E = nullptr) {
    if (!ctx->have_bcomm) return BTE_OK;
    std::string e;
    if (!bte::nccl::allreduce_sum_f64(ctx->bcomm, E ? E : ctx->E, ctx->nc, ctx->stream, &e)) {
        set_err(&ctx->err, "NCCL all-reduce failed: %s", e.c_str());
        return BTE_ENCCL;
    }
    return BTE_OK;
}

bte_status reduce_slots(bte_ctx *ctx) {
    const int tb = 256;
    bte::sum_slots_kernel<<<(ctx->nc + tb - 1) / tb, tb, 0, ctx->stream>>>(ctx->part, ctx->n_slots_step, ctx->nc,
                                                                           ctx->E, ctx->d_halt);
    ctx->st.kernel_launches++;
    CUDA_TRY(ctx, cudaGetLastError());
    return BTE_OK;
}

// Band-sharded step exchange (SURVEY 8(e) alternative, no replicated solve):
// E (slot sum, padded to world x chunk) -> reduce-scatter -> Newton on this
// rank's chunk of cells -> all-gather of T -> every rank finishes its rows.
bte_status shard_newton_step(bte_ctx *ctx) {
    std::string e;
    ev_mark(ctx, kPhAllreduce, true);
    STATUS_TRY(reduce_slots(ctx));
    if (!bte::nccl::reduce_scatter_sum_f64(ctx->bcomm, ctx->E, ctx->Echunk, ctx->chunk, ctx->stream, &e))
        return set_err(&ctx->err, "NCCL reduce-scatter failed: %s", e.c_str()), BTE_ENCCL;
    ev_mark(ctx, kPhAllreduce, false);
    ev_mark(ctx, kPhNewton, true);
    bte::NewtonParams q = newton_params(ctx, ctx->Echunk, /*step=*/true);
    q.c_lo = ctx->gband * ctx->chunk;
    q.nc = std::max(0, std::min(ctx->chunk, ctx->nc - q.c_lo));
    q.T_out = ctx->Tg;
    q.neg_fail = 1;
    if (warp_newton(ctx, q.nc)) STATUS_TRY(launch_newton_warp(ctx, q));
    else STATUS_TRY(launch_newton_cells(ctx, q));
    double *mine = ctx->Tg + (size_t)ctx->gband * ctx->chunk;
    if (!bte::nccl::allgather_f64(ctx->bcomm, mine, ctx->Tg, ctx->chunk, ctx->stream, &e))
        return set_err(&ctx->err, "NCCL all-gather failed: %s", e.c_str()), BTE_ENCCL;
    STATUS_TRY(newton_finish(ctx));
    ev_mark(ctx, kPhNewton, false);
    if (ctx->td) ctx->rsel = 1 - ctx->rsel;
    CUDA_TRY(ctx, cudaGetLastError());
    return BTE_OK;
}

// ------------------------------------------------------------- halo (N3)
// Pack / unpack one segment for every local band-row (current slabs).
bte::HaloParams halo_params(const bte_ctx *ctx) {
    bte::HaloParams hp{};
    for (int k = 0; k < ctx->nb_loc; ++k) hp.row[k] = ctx->pool_cells + (int64_t)ctx->cur_slot[k] * ctx->slab_elems;
    hp.nb_loc = ctx->nb_loc;
    hp.ps = ctx->ps;
    hp.fail = ctx->d_fail;
    return hp;
}

dim3 halo_grid(const bte_ctx *ctx, int64_t per) {
    return dim3((unsigned)std::max<int64_t>(1, std::min<int64_t>(2048, (per + 255) / 256)), (unsigned)ctx->nb_loc);
}

bte_status halo_pack(bte_ctx *ctx, const HaloSeg &h) {
    if (h.n_send() == 0) return BTE_OK;
    bte::HaloParams hp = halo_params(ctx);
    hp.cells = h.send_cells;
    hp.dirs = h.send_dirs;
    hp.n = h.n_send_cells;
    hp.n_dirs = h.n_send_dirs;
    bte::halo_pack_kernel<<<halo_grid(ctx, h.n_send()), 256, 0, ctx->stream>>>(hp, h.sbuf);
    ctx->st.kernel_launches++;
    CUDA_TRY(ctx, cudaGetLastError());
    return BTE_OK;
}

bte_status halo_unpack(bte_ctx *ctx, const HaloSeg &h) {
    if (h.n_recv() == 0) return BTE_OK;
    bte::HaloParams hp = halo_params(ctx);
    hp.dirs = h.recv_dirs;
    hp.n = h.n_recv_cells;
    hp.n_dirs = h.n_recv_dirs;
    hp.cells = h.recv_cols;
    bte::halo_unpack_kernel<<<halo_grid(ctx, h.n_recv()), 256, 0, ctx->stream>>>(hp, h.rbuf);
    ctx->st.kernel_launches++;
    CUDA_TRY(ctx, cudaGetLastError());
    return BTE_OK;
}

// Cell-partitioned step, before the flux: every segment packed, one NCCL group
// of sends / receives with the neighbour parts of this band group, unpacked
// into the halo columns of the current slabs (I^n, the old level, Eq. 3).
bte_status halo_exchange(bte_ctx *ctx) {
    if (ctx->hsegs.empty()) return BTE_OK;
    if (!ctx->have_comm) return set_err(&ctx->err, "halo exchange needs a communicator"), BTE_ESTATE;
    ev_mark(ctx, kPhHalo, true);
    for (const HaloSeg &h : ctx->hsegs) STATUS_TRY(halo_pack(ctx, h));
    std::vector<bte::nccl::P2P> ops;
    for (const HaloSeg &h : ctx->hsegs)
        ops.push_back({ctx->gband * ctx->n_parts + h.part, h.sbuf, h.n_send() * ctx->nb_loc, h.rbuf,
                       h.n_recv() * ctx->nb_loc});
    std::string e;
    if (!bte::nccl::exchange_f64(ctx->comm, ops.data(), (int)ops.size(), ctx->stream, &e))
        return set_err(&ctx->err, "NCCL halo exchange failed: %s", e.c_str()), BTE_ENCCL;
    for (const HaloSeg &h : ctx->hsegs) STATUS_TRY(halo_unpack(ctx, h));
    ev_mark(ctx, kPhHalo, false);
    return BTE_OK;
}


// T <- Tg (a negative entry marks a failed cell: flag, keep T^n), Tr <- T^n,
// I0 and the rate table of the local rows at the new T.
bte_status newton_finish(bte_ctx *ctx) {
    bte::newton_finish_kernel<<<(ctx->nc + 255) / 256, 256, 0, ctx->stream>>>(
        ctx->Tg, ctx->T, ctx->nc, ctx->b_lo, ctx->nb_loc, ctx->Cb, ctx->theta, ctx->i0, ctx->td, ctx->d_ra, ctx->d_rb,
        ctx->d_rth, ctx->Tr, ctx->td ? rate_half(ctx, ctx->rsel) : nullptr, ctx->d_fail, ctx->d_halt, ctx->d_done);
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
    if (ctx->td) ctx->rsel = 1 - ctx->rsel;
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

// ------------------------------------------------------------- z-slab partitions of box grids
// A cell partition of a structured 3-D box grid into slabs of whole grid
// axis-2 layers (each part a contiguous layer range) keeps the box kernel: the
// rank's slab tensor holds its owned layers plus the neighbour parts' adjacent
// layer (halo) below / above, the kernel updates the owned layers only and
// takes the upwind layer of a range from the halo layer exactly as from a
// neighbouring range (Eq. 3); the global walls stay wall ghosts (Eq. 6).
struct ZSlab {
    bool on = false;
    int32_t za = 0, zb = 0, h_lo = 0, h_hi = 0;
    int64_t off = 0;                // columns before the first owned cell (the lower halo layer)
    BoxDetect gbx;                  // the global box
    std::vector<bte::BoxOrbit> orbs;
    std::vector<int64_t> grid_of;   // global cell -> grid lexicographic position
};

ZSlab detect_zslab(const bte_mesh *m, const bte_dirs *dr, const bte_bcs *bc, const bte_options *o, int me) {
    ZSlab z;
    if (m->dim != 3 || (o->flags & (BTE_FLAG_NO_BOX | BTE_FLAG_NO_TMA | BTE_FLAG_GENERIC_FACES)))
        return z;
    z.gbx = detect_box(m, bc);
    const BoxDetect &g = z.gbx;
    if (!g.ok || !box_orbits(dr, g.ax, g.zside[0] == 1 || g.zside[1] == 1, &z.orbs)) return z;
    const int64_t plane = (int64_t)g.n[0] * g.n[1];
    std::vector<int32_t> layer_part(g.n[2], -1);
    for (int32_t l = 0; l < g.n[2]; ++l)
        for (int64_t i = 0; i < plane; ++i) {
            const int32_t pp = o->cell_part[g.cell_at[l * plane + i]];
            if (pp < 0 || pp >= o->n_cell_parts) return z;
            if (layer_part[l] < 0) layer_part[l] = pp;
            else if (layer_part[l] != pp) return z;  // a layer split between parts
        }
    int32_t za = -1, zb = -1;
    for (int32_t l = 0; l < g.n[2]; ++l)
        if (layer_part[l] == me) {
            if (za < 0) za = l;
            else if (zb != l) return z;  // not contiguous
            zb = l + 1;
        }
    if (za < 0) return z;
    z.za = za;
    z.zb = zb;
    z.h_lo = za > 0;
    z.h_hi = zb < g.n[2];
    z.off = z.h_lo * plane;
    z.grid_of.assign(m->n_cells, -1);
    for (int64_t i = 0; i < (int64_t)g.cell_at.size(); ++i) z.grid_of[g.cell_at[i]] = i;
    z.on = true;
    return z;
}

// ------------------------------------------------------------- cell partition (N3)
// The owned cells of part `me` as a mesh of their own: owned cells in ascending
// global id (local ids 0..nc-1), faces copied in stored order; a face whose
// neighbour lies in another part points to a halo column nc + slot (the slots
// of one neighbour part contiguous, ascending global id).  Segments (one per
// neighbour part): cells and directions follow the READING
// side's faces (a cut face f of a reader cell needs the writer's value for the
// directions with s_d . n_f < 0, the upwind inflow of Eq. 3), so both ends of
// a segment derive the same lists from the replicated global mesh.
struct SegPlan {
    int part = 0;
    std::vector<int32_t> send_local, send_dirs, recv_dirs;
    std::vector<int64_t> recv_global;  // the halo cells (global ids, ascending)
    int32_t n_recv_cells = 0, col0 = 0;
};
struct LocalPlan {
    std::vector<int64_t> gid, off, nbr;
    std::vector<double> area, nrm, vol, cen;
    std::vector<SegPlan> segs;
    int32_t n_halo = 0;
    bte_mesh mesh{};
};

bte_status build_local(const bte_mesh *m, const bte_dirs *dr, const bte_options *o, int me, LocalPlan *L) {
    const int64_t N = m->n_cells;
    const int P = o->n_cell_parts;
    const int32_t *part = o->cell_part;
    for (int64_t c = 0; c < N; ++c)
        if (part[c] < 0 || part[c] >= P)
            return set_err(nullptr, "cell_part[%lld] = %d outside [0, %d)", (long long)c, part[c], P), BTE_EINVAL;
    std::vector<int64_t> loc(N, -1);
    for (int64_t c = 0; c < N; ++c)
        if (part[c] == me) loc[c] = (int64_t)L->gid.size(), L->gid.push_back(c);
    if (L->gid.empty()) return set_err(nullptr, "cell part %d has no cells", me), BTE_EINVAL;
    std::vector<std::vector<int64_t>> rc(P), sc(P);
    std::vector<std::set<std::array<double, 3>>> rn(P), sn(P);
    for (int64_t g = 0; g < N; ++g) {
        const int pg = part[g];
        for (int64_t f = m->face_offsets[g]; f < m->face_offsets[g + 1]; ++f) {
            const int64_t h = m->face_nbr[f];
            if (h < 0 || part[h] == pg) continue;
            const std::array<double, 3> n = {m->face_normal[3 * f], m->face_normal[3 * f + 1], m->face_normal[3 * f + 2]};
            if (pg == me) rc[part[h]].push_back(h), rn[part[h]].insert(n);  // g reads h
            if (part[h] == me) sc[pg].push_back(h), sn[pg].insert(n);       // h is read by g
        }
    }
    auto dirs_of = [&](const std::set<std::array<double, 3>> &ns) {
        std::vector<int32_t> out;
        for (int d = 0; d < dr->n_dirs; ++d) {
            const double *s = dr->s + 3 * d;
            for (const auto &n : ns)
                if (s[0] * n[0] + s[1] * n[1] + s[2] * n[2] < 0.0) {
                    out.push_back(d);
                    break;
                }
        }
        return out;
    };
    std::vector<int32_t> hslot(N, -1);
    for (int q = 0; q < P; ++q) {
        if (q == me) continue;
        auto uniq = [](std::vector<int64_t> &v) {
            std::sort(v.begin(), v.end());
            v.erase(std::unique(v.begin(), v.end()), v.end());
        };
        uniq(rc[q]);
        uniq(sc[q]);
        if (rc[q].empty() && sc[q].empty()) continue;
        SegPlan s;
        s.part = q;
        s.col0 = L->n_halo;
        for (int64_t h : rc[q]) hslot[h] = L->n_halo++;
        s.n_recv_cells = (int32_t)rc[q].size();
        s.recv_global = rc[q];
        s.recv_dirs = dirs_of(rn[q]);
        for (int64_t h : sc[q]) s.send_local.push_back((int32_t)loc[h]);
        s.send_dirs = dirs_of(sn[q]);
        L->segs.push_back(std::move(s));
    }
    const int64_t nc = (int64_t)L->gid.size();
    L->off.push_back(0);
    for (int64_t i = 0; i < nc; ++i) {
        const int64_t c = L->gid[i];
        for (int64_t f = m->face_offsets[c]; f < m->face_offsets[c + 1]; ++f) {
            const int64_t h = m->face_nbr[f];
            L->nbr.push_back(h < 0 ? h : part[h] == me ? loc[h] : nc + hslot[h]);
            L->area.push_back(m->face_area[f]);
            for (int a = 0; a < 3; ++a) L->nrm.push_back(m->face_normal[3 * f + a]);
        }
        L->off.push_back((int64_t)L->nbr.size());
        L->vol.push_back(m->cell_volume[c]);
        if (m->cell_centre)
            for (int a = 0; a < 3; ++a) L->cen.push_back(m->cell_centre[3 * c + a]);
    }
    L->mesh.dim = m->dim;
    L->mesh.n_cells = nc;
    L->mesh.face_offsets = L->off.data();
    L->mesh.face_nbr = L->nbr.data();
    L->mesh.face_area = L->area.data();
    L->mesh.face_normal = L->nrm.data();
    L->mesh.cell_volume = L->vol.data();
    L->mesh.cell_centre = m->cell_centre ? L->cen.data() : nullptr;
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
                    ctx->d_iter_max, ctx->d_flags, ctx->d_smax, ctx->orb, ctx->dirs_box, ctx->side_tab, ctx->side_col,
                    ctx->d_ra, ctx->d_rb, ctx->d_rth, ctx->d_inv_v, ctx->rates, ctx->Tr,
                    ctx->E2, ctx->T2, ctx->cw_diag, ctx->Echunk, ctx->Tg, ctx->hl_off, ctx->hl_cell, ctx->sidx, ctx->bl_off, ctx->bl_col, ctx->bl_cls};
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
    if (const char *ev = std::getenv("BTE_NEWTON"))
        ctx->newton_mode = std::strcmp(ev, "warp") == 0 ? 1 : std::strcmp(ev, "thread") == 0 ? 2 : 0;
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
        // shared memory for 2 CTAs per SM: ring stages x 12 KB + 16 KB output + L x 2 KB energy
        // (rate law: 16 KB stages; 5 stages x 4 layers fit twice per SM, measured best)
        const char *ev = std::getenv("BTE_BOX_STAGES");
        // (2-D, 3 CTAs per SM: 4 stages, 3 with the rate rows; orbit chunks of 25 (a C3 slice = 4 chunks))
        const int def_stages = bx.flat ? (td ? 3 : 4) : (td ? 5 : 6);
        ctx->box_stages = std::max(2, std::min(bte::kBoxMaxStages, ev ? std::atoi(ev) : def_stages));
        if (bx.flat) ctx->box_oc = 25;
        ev = std::getenv("BTE_BOX_L");
        ctx->box_L = std::max(1, std::min<int>(bx.n[2], ev ? std::atoi(ev) : (td ? 4 : 8)));
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
        const size_t reserve = (size_t)1 << 30;
        while (n_spare > 1 && (size_t)(nb_loc + n_spare) * slab_bytes + other + reserve > free_b) --n_spare;
        if ((size_t)(nb_loc + n_spare) * slab_bytes + other > free_b) {
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

    const int max_slots = count_slots(ctx);
    CREATE_TRY(dalloc(ctx, &ctx->part, (size_t)max_slots * nc));
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
        // per tile: own cells [0, 256), halo cells (interior faces pointing out of the
        // tile) [256, 256 + nh), boundary-face ghosts [256 + nh, 256 + nh + ng)
        const int32_t ntiles = (nc + bte::kTile - 1) / bte::kTile;
        std::vector<int32_t> hoff(ntiles + 1, 0), hcell, goff(ntiles + 1, 0), gcol, gcls;
        std::vector<uint16_t> sidx_h(ell, 0);
        int32_t smax = 0;
        std::map<int32_t, int32_t> slot_of;
        std::vector<size_t> bq;
        for (int32_t t = 0; t < ntiles; ++t) {
            const int32_t t0 = t * bte::kTile, t1 = std::min(nc, t0 + bte::kTile);
            slot_of.clear();
            bq.clear();
            for (int j = 0; j < mf_t; ++j)
                for (int32_t i = t0; i < t1; ++i) {
                    const size_t q = (size_t)j * nc + i;
                    if (fcode8_h[q] != bte::kCode8Interior) {
                        bq.push_back(q);
                        continue;
                    }
                    const int32_t v = nbr_h[q];
                    if (v >= t0 && v < t0 + bte::kTile) {
                        sidx_h[q] = (uint16_t)(v - t0);
                    } else {
                        auto it = slot_of.find(v);
                        if (it == slot_of.end()) it = slot_of.emplace(v, (int32_t)slot_of.size()).first;
                        sidx_h[q] = (uint16_t)(bte::kTile + it->second);
                    }
                }
            const int32_t nh = (int32_t)slot_of.size();
            std::vector<int32_t> cells(nh);
            for (const auto &kv : slot_of) cells[kv.second] = kv.first;
            hcell.insert(hcell.end(), cells.begin(), cells.end());
            hoff[t + 1] = (int32_t)hcell.size();
            for (size_t g = 0; g < bq.size(); ++g) {  // Eq. 6 ghosts: isothermal table column / reflected plane
                const size_t q = bq[g];
                const int32_t i = (int32_t)(q % (size_t)nc);
                const bool iso = fcode8_h[q] == bte::kCode8Iso;
                gcol.push_back(iso ? nbr_h[q] : i);
                gcls.push_back(iso ? -1 : (int32_t)fcode8_h[q]);
                sidx_h[q] = (uint16_t)(bte::kTile + nh + (int32_t)g);
            }
            goff[t + 1] = (int32_t)gcol.size();
            smax = std::max<int32_t>(smax, nh + (int32_t)bq.size());
        }
        if (smax <= bte::kMaxTileStaged) {
            ctx->hstride = bte::kTile + (smax + 31) / 32 * 32;
            CREATE_TRY(upload(ctx, &ctx->hl_off, hoff));
            CREATE_TRY(upload(ctx, &ctx->hl_cell, hcell));
            CREATE_TRY(upload(ctx, &ctx->bl_off, goff));
            CREATE_TRY(upload(ctx, &ctx->bl_col, gcol));
            CREATE_TRY(upload(ctx, &ctx->bl_cls, gcls));
            CREATE_TRY(upload(ctx, &ctx->sidx, sidx_h));
        } else {
            ctx->tma = false;  // too much to stage per tile: the register kernel
        }
    }
    CREATE_TRY(upload(ctx, &ctx->d_cur_slot, ctx->cur_slot));
    CREATE_TRY(upload(ctx, &ctx->nbr, nbr_h));
    CREATE_TRY(upload(ctx, &ctx->nbm, nbm_h));
    CREATE_TRY(upload(ctx, &ctx->fcode, fcode_h));
    CREATE_TRY(upload(ctx, &ctx->fcode8, fcode8_h));
    CREATE_TRY(upload(ctx, &ctx->gx, gx_h));
    CREATE_TRY(upload(ctx, &ctx->gy, gy_h));
    CREATE_TRY(upload(ctx, &ctx->gz, gz_h));
    CREATE_TRY(upload(ctx, &ctx->pos, pos_h));
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
    CREATE_TRY(upload(ctx, &ctx->cw_all, cw));
    CREATE_TRY(dalloc(ctx, &ctx->i0w, (size_t)nb_loc * std::max(1, ctx->n_iso)));
    CREATE_TRY(dalloc(ctx, &ctx->d_iter_max, 1));
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

// With the rate law the bound depends on the hottest temperature the state can
// reach (t_hi); under cell partitioning each rank only sees its own cells, so
// the ranks agree on the max first (every bte_step of such a run is collective
// anyway), and all of them accept or reject the same dt.
static bte_status sync_dt_bound(bte_ctx *ctx) {
    if (!(ctx->td && ctx->n_parts > 1 && ctx->have_comm)) return BTE_OK;
    double *d = reinterpret_cast<double *>(ctx->d_smax);
    CUDA_TRY(ctx, cudaMemcpyAsync(d, &ctx->t_hi, sizeof(double), cudaMemcpyHostToDevice, ctx->stream));
    std::string e;
    if (!bte::nccl::allreduce_max_f64(ctx->comm, d, 1, ctx->stream, &e))
        return set_err(&ctx->err, "all-reduce (max) of the hottest temperature failed: %s", e.c_str()), BTE_ENCCL;
    CUDA_TRY(ctx, cudaMemcpyAsync(&ctx->t_hi, d, sizeof(double), cudaMemcpyDeviceToHost, ctx->stream));
    CUDA_TRY(ctx, cudaStreamSynchronize(ctx->stream));
    update_dt_bound(ctx);
    return BTE_OK;
}

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

// rows of nc doubles (device rows of `stride` elements, internal order) <-> host (caller order)
static bte_status rows_to_host(const bte_ctx *cctx, const double *dsrc, int64_t stride, int64_t rows, double *host) {
    bte_ctx *ctx = const_cast<bte_ctx *>(cctx);
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
    const int tb = 128;
    const bool law_r2 = ctx->td && ctx->opt.temp_rule == 0;  // weights at the kept rate temperature
    bte::energy_kernel<<<(ctx->nc + tb - 1) / tb, tb, 0, ctx->stream>>>(
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
    const int tb = 128;
    bte::energy_kernel<<<(ctx->nc + tb - 1) / tb, tb, 0, ctx->stream>>>(
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

bte_status bte_local_cells(const bte_ctx *ctx, int64_t *n_local, int64_t *ids) {
    if (!ctx || !n_local) return BTE_EINVAL;
    *n_local = ctx->nc;
    if (ids)
        for (int32_t i = 0; i < ctx->nc; ++i) ids[i] = ctx->gid.empty() ? i : ctx->gid[i];
    return BTE_OK;
}

static const HaloSeg *find_seg(const bte_ctx *ctx, int32_t part, bte_status *st) {
    *st = BTE_OK;
    if (part < 0 || part >= ctx->n_parts) {
        set_err(const_cast<std::string *>(&ctx->err), "part %d outside [0, %d)", part, ctx->n_parts);
        *st = BTE_EINVAL;
        return nullptr;
    }
    for (const HaloSeg &h : ctx->hsegs)
        if (h.part == part) return &h;
    return nullptr;  // no shared face: empty segment
}

bte_status bte_halo_size(const bte_ctx *ctx, int32_t part, int64_t *n_send, int64_t *n_recv) {
    if (!ctx || !n_send || !n_recv) return BTE_EINVAL;
    bte_status st;
    const HaloSeg *h = find_seg(ctx, part, &st);
    STATUS_TRY(st);
    *n_send = h ? h->n_send() * ctx->nb_loc : 0;
    *n_recv = h ? h->n_recv() * ctx->nb_loc : 0;
    return BTE_OK;
}

bte_status bte_halo_export(const bte_ctx *cctx, int32_t part, double *buf) {
    if (!cctx || !buf) return BTE_EINVAL;
    bte_ctx *ctx = const_cast<bte_ctx *>(cctx);
    if (ctx->begun) return set_err(&ctx->err, "split step in flight"), BTE_ESTATE;
    bte_status st;
    const HaloSeg *h = find_seg(ctx, part, &st);
    STATUS_TRY(st);
    if (!h || h->n_send() == 0) return BTE_OK;
    CUDA_TRY(ctx, cudaSetDevice(ctx->device));
    STATUS_TRY(halo_pack(ctx, *h));
    CUDA_TRY(ctx, cudaMemcpyAsync(buf, h->sbuf, (size_t)h->n_send() * ctx->nb_loc * sizeof(double),
                                  cudaMemcpyDeviceToHost, ctx->stream));
    CUDA_TRY(ctx, cudaStreamSynchronize(ctx->stream));
    return BTE_OK;
}

bte_status bte_halo_import(bte_ctx *ctx, int32_t part, const double *buf) {
    if (!ctx || !buf) return BTE_EINVAL;
    if (ctx->begun) return set_err(&ctx->err, "split step in flight"), BTE_ESTATE;
    bte_status st;
    const HaloSeg *h = find_seg(ctx, part, &st);
    STATUS_TRY(st);
    if (!h || h->n_recv() == 0) return BTE_OK;
    CUDA_TRY(ctx, cudaSetDevice(ctx->device));
    CUDA_TRY(ctx, cudaMemcpyAsync(h->rbuf, buf, (size_t)h->n_recv() * ctx->nb_loc * sizeof(double),
                                  cudaMemcpyHostToDevice, ctx->stream));
    STATUS_TRY(halo_unpack(ctx, *h));
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
