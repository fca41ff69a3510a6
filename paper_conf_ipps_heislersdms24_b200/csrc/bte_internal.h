// bte_internal.h -- the library's internal state (struct bte_ctx) and the
// functions the host units share.  Not part of the ABI (include/bte.h is).
//
// Units (all host code; the arithmetic of the step is in the kernels):
//   bte_create.cu  validation, structure detection (box grids, z slabs, cell
//                  partitions), device layout, bte_create / bte_destroy
//   bte_plan.cu    launch planning: flux-kernel dispatch, box work items,
//                  energy slots, shared-memory opt-ins
//   bte_step.cu    the step: flux launches, temperature solve, failure stop,
//                  CUDA-graph replay, bte_step / split step
//   bte_dist.cu    multi-rank exchanges: energy reduce-scatter / all-gather /
//                  all-reduce, halo exchange, cell-partition ABI
//   bte_state.cu   getters / setters / re-solves / stats
#pragma once
#include "../../include/bte.h"
#include "bte_kernels.cuh"
#include "bte_nccl.h"

#include <cudaTypedefs.h>  // PFN_cuTensorMapEncodeTiled (driver entry point, no -lcuda)

#include <algorithm>
#include <array>
#include <cmath>
#include <cstdarg>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>
#include <vector>

namespace bte_host {

// CODATA 2018 values (the library's own copy; theta_b = hbar omega_b / kB).
constexpr double kHbar = 1.054571817e-34;
constexpr double kKb = 1.380649e-23;
constexpr int kMaxFaces = 8;

extern thread_local std::string g_err;  // last error of this thread (bte_last_error(NULL))
void set_err(std::string *dst, const char *fmt, ...);


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

}  // namespace bte_host

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
    bool identity_order = false;  // internal cell order == the caller's (pos[i] == i): no gather / scatter
    uint32_t *fcode = nullptr;  // paired: 5-bit face codes per cell
    uint8_t *fcode8 = nullptr;  // generic: 8-bit face codes per face slot
    double *gx = nullptr, *gy = nullptr, *gz = nullptr;
    bool paired = false;     // every cell's faces are exact opposite pairs
    bool uniform_g = false;  // ... and every cell has the same g per pair
    bool tma = false;        // 256-thread blocks: the TMA-staged kernel (paired or generic faces)
    int32_t *hl_off = nullptr, *hl_cell = nullptr, *hl_pos = nullptr;  // generic TMA kernel: per-tile halo lists,
    int32_t *bl_off = nullptr, *bl_col = nullptr, *bl_cls = nullptr, *bl_pos = nullptr;  // ... ghost lists
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
    bool rate_now = false;  // ... of the step's own T (reading 26; else lagged one step, reading 22)
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
    // terms of the temperature equation with constant weights: rows with the same
    // theta (the LA and TA rows of a band) share one expm1; K_j = sum c_b C_b
    int n_terms = 0;
    double *t_th = nullptr, *t_k = nullptr, *t_ic = nullptr;  // theta_j, K_j, 1 / C of the representative row
    int32_t *t_rep = nullptr;                                  // representative row (the I0 table of T^n)
    int32_t *t_nrow = nullptr;                                 // [nb] next row of the same term (-1: none)
    int8_t *fresh = nullptr;                                   // [nc] I0 stored by the step's solve (lanes path)
    int32_t *d_iter_max = nullptr;
    // d_flags[0] fail (a temperature solve failed), [1] halt (the fail flag as the
    // step's flux launch saw it: the rest of the step is a no-op), [2] steps done
    // (counted by each step's last kernel; the host undoes the slab rotation of
    // the steps skipped after a failure, so the state is that of the failing step)
    int32_t *d_flags = nullptr, *d_fail = nullptr, *d_halt = nullptr, *d_done = nullptr;
    int32_t done_seen = 0;
    int newton_mode = 0;  // the step's solve: 0 by mesh size, 2 thread per cell, 4/8/16/32 lanes per cell
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
    std::vector<bte_host::HaloSeg> hsegs;
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
    std::vector<bte_host::PhaseEvent> ev_live, ev_pool;
};

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


namespace bte_host {

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

// ---- bte_layout.cu
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

BoxDetect detect_box2d(const bte_mesh *m, const bte_bcs *bc);
BoxDetect detect_box(const bte_mesh *m, const bte_bcs *bc);
bool box_orbits(const bte_dirs *dr, const int ax[3], bool need_rz, std::vector<bte::BoxOrbit> *out);
bool encode_map(CUtensorMap *tm, void *base, int rank, const uint64_t *dims, const uint64_t *strides,
                const uint32_t *box);
ZSlab detect_zslab(const bte_mesh *m, const bte_dirs *dr, const bte_bcs *bc, const bte_options *o, int me);
bte_status build_local(const bte_mesh *m, const bte_dirs *dr, const bte_options *o, int me, LocalPlan *L);

// ---- bte_plan.cu
cudaError_t ensure_smem(const void *fn, size_t smem);
using FluxLaunch = cudaError_t (*)(dim3, dim3, cudaStream_t, const bte::FluxParams &);
FluxLaunch pick_flux(int dim, int mf_t, int bg, bool paired, bool uniform_g, bool tma);
int legal_bg(int bg, bool paired);
struct BoxPlan {
    int tiles0, tiles1, zranges, n_batches, n_chunks, nbb, oc;
};
BoxPlan plan_box(const bte_ctx *ctx, int nbl);
int box_stage(const bte_ctx *ctx);
size_t box_smem(const bte_ctx *ctx);
using BoxKernel = void (*)(const bte::BoxParams, const CUtensorMap, const CUtensorMap, const CUtensorMap,
                           const CUtensorMap, const CUtensorMap);
BoxKernel box_kernel(const bte_ctx *ctx);
bte_status box_setup_kernel(bte_ctx *ctx);
double *rate_half(bte_ctx *ctx, int sel);
struct LaunchPlan {
    int groups, n_dch, dchunk;
};
struct Segment {
    int off, nbl, bg;
};
std::vector<Segment> segments(const bte_ctx *ctx, int nbl);
LaunchPlan plan_launch(const bte_ctx *ctx, int nbl, int bg);
int count_slots(const bte_ctx *ctx);

// ---- bte_step.cu
void ev_mark(bte_ctx *ctx, int phase, bool begin);
void ev_collect(bte_ctx *ctx);
bte_status run_flux(bte_ctx *ctx, double dt);
bool warp_newton(const bte_ctx *ctx, int ncells);
bte_status launch_newton_cells(bte_ctx *ctx, const bte::NewtonParams &q);
bte_status launch_newton_warp(bte_ctx *ctx, const bte::NewtonParams &q);
bte::NewtonParams newton_params(bte_ctx *ctx, const double *E_or_null, bool step);
bte_status run_newton(bte_ctx *ctx, const double *E_or_null, bool step = true);
bte_status newton_finish(bte_ctx *ctx, const int8_t *fresh = nullptr);
bte_status reduce_slots(bte_ctx *ctx);
bte_status read_flags(bte_ctx *ctx, bool *failed, int64_t *ran);
bte_status check_newton(bte_ctx *ctx);
void undo_step_rotation(bte_ctx *ctx);
bte_status refresh_i0(bte_ctx *ctx);
void update_dt_bound(bte_ctx *ctx);
bte_status upload_cur_slots(bte_ctx *ctx);

// ---- bte_dist.cu
bte_status allreduce_E(bte_ctx *ctx, double *E = nullptr);
bte_status shard_newton_step(bte_ctx *ctx);
bte_status halo_pack(bte_ctx *ctx, const HaloSeg &h);
bte_status halo_unpack(bte_ctx *ctx, const HaloSeg &h);
bte_status halo_exchange(bte_ctx *ctx);
bte_status sync_dt_bound(bte_ctx *ctx);

}  // namespace bte_host
