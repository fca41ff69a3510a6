// bte_plan.cu -- launch planning (see bte_internal.h): which flux kernel and
// band group a launch uses, the box kernel's work items (band-rows x orbit
// chunk x 32 x 8 x L cells per CTA), the energy-partial slots of a step, and
// the shared-memory opt-ins of the kernels.
#include "bte_internal.h"
#include <map>
#include <mutex>

namespace bte_host {


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
template <int DIM, int MF, int BG, bool TD, int HS>
cudaError_t flux_tma_generic_launch_hs(dim3 g, const bte::FluxParams &p, cudaStream_t s) {
    const size_t smem = (size_t)bte::kStagesG * BG * p.hstride * sizeof(double) + (size_t)p.dchunk * sizeof(double4) +
                        3 * (size_t)(p.hstride - bte::kTile) * sizeof(int32_t);  // (+ the tile's staging lists)
    cudaError_t e = ensure_smem((const void *)bte::flux_tma_generic_kernel<DIM, MF, BG, TD, HS>, smem);
    if (e != cudaSuccess) return e;
    bte::flux_tma_generic_kernel<DIM, MF, BG, TD, HS><<<g, dim3(bte::kTmaThreads), smem, s>>>(p);
    return cudaGetLastError();
}
// (the staged row stride of the common case as a compile-time constant)
template <int DIM, int MF, int BG, bool TD>
cudaError_t flux_tma_generic_launch_td(dim3 g, const bte::FluxParams &p, cudaStream_t s) {
    if (p.hstride == bte::kTileStagedFixed) return flux_tma_generic_launch_hs<DIM, MF, BG, TD, bte::kTileStagedFixed>(g, p, s);
    return flux_tma_generic_launch_hs<DIM, MF, BG, TD, 0>(g, p, s);
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
    const size_t obuf = (ctx->bflat ? bte::box_obuf<true>() : bte::box_obuf<false>())
                            ? 2 * 4 * bte::kBoxCells  // double-buffered output tiles of the tensor stores
                            : 0;                      // results leave straight from registers
    return ((size_t)ctx->box_stages * stage + obuf + (size_t)ctx->box_L * bte::kBoxCells) *
               sizeof(double) +
           (size_t)kBoxMaxOrbChunk * sizeof(bte::BoxOrbitC);
}
BoxKernel box_kernel(const bte_ctx *ctx) {
    if (ctx->bflat) return ctx->td ? bte::flux_box_kernel<true, true> : bte::flux_box_kernel<false, true>;
    return ctx->td ? bte::flux_box_kernel<true, false> : bte::flux_box_kernel<false, false>;
}

bte_status box_setup_kernel(bte_ctx *ctx) {
    const size_t smem = box_smem(ctx);
    CUDA_TRY(ctx, ensure_smem((const void *)box_kernel(ctx), smem));  // (per device, raised only)
    int occ = 0;
    CUDA_TRY(ctx, cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, box_kernel(ctx), bte::kBoxThreads, smem));
    ctx->box_ctas_per_sm = std::max(1, occ);
    return BTE_OK;
}

// Rate tables (N1): half `sel` of ctx->rates.
double *rate_half(bte_ctx *ctx, int sel) { return ctx->rates + (size_t)sel * ctx->nb_loc * ctx->nc; }
// Launches of a batch of nbl band-rows: groups of bg rows (bg a power of two for
// generic faces).  The TMA-staged generic-face kernel takes a ragged last group
// (one launch: C3t's 55 rows were 52 + 2 + 1 in three launches, 1.77 -> ~1.7 ms);
// the others launch the remainder with smaller groups.
std::vector<Segment> segments(const bte_ctx *ctx, int nbl) {
    const int bg = ctx->bg;
    const bool paired = ctx->paired;
    if (ctx->tma && !paired) return {{0, nbl, bg}};
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
    lp.groups = (nbl + bg - 1) / bg;  // (a ragged last group: the generic TMA kernel)
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
        for (const Segment &sg : segments(ctx, std::min(ctx->n_spare, ctx->nb_loc - l0))) {
            const LaunchPlan lp = plan_launch(ctx, sg.nbl, sg.bg);
            slots += lp.groups * lp.n_dch;
        }
    return slots;
}

}  // namespace bte_host
