// bte_staging.h -- host-side layout of the generic-face TMA kernel's shared-memory
// stage (bte_create): bank-conflict-aware positions of a tile's halo cells and
// ghosts, and the per-cell order of face slots.  Plain C++ (no CUDA): the CPU
// tests compile it on its own (tests/test_staging_host.py).
#pragma once
#include <algorithm>
#include <array>
#include <climits>
#include <cstdint>
#include <cstring>
#include <utility>
#include <vector>

namespace bte_host {

// Shared-memory bank conflicts of the generic TMA kernel.  A warp reads face
// slot j's upwind values with one 64-bit shared load per band-row, at the staged
// indices sidx[j][lane]; the hardware serves each half-warp (16 lanes) in as many
// wavefronts as the most distinct values that share a bank pair (index mod 16),
// equal values broadcast (measured on B200: C3t 4.5 wavefronts per warp load
// before, ncu, against 2 without conflicts).
// cnt[k] = distinct values of v[0..n) in bank class k.
// (staged indices are < 1024: kTile + kMaxTileStaged; a 1024-bit set marks the seen ones)
inline void class_counts(const uint16_t *v, int n, int cnt[16]) {
    uint64_t seen[16] = {};
    for (int k = 0; k < 16; ++k) cnt[k] = 0;
    for (int a = 0; a < n; ++a) {
        const uint32_t x = v[a];
        uint64_t &w = seen[(x >> 6) & 15];
        const uint64_t bit = 1ull << (x & 63);
        if (!(w & bit)) {
            w |= bit;
            ++cnt[x & 15];
        }
    }
}
// Wavefronts of a half-warp's loads of every slot (cost) and a smooth version
// that also rewards evenly spread classes (the local search's objective).
inline void half_costs(const uint16_t (*col)[16], int mf, int n, int *wave, int *smooth) {
    int w = 0, sm = 0, cnt[16];
    for (int j = 0; j < mf; ++j) {
        class_counts(col[j], n, cnt);
        int mx = 0;
        for (int k = 0; k < 16; ++k) {
            mx = std::max(mx, cnt[k]);
            sm += cnt[k] * cnt[k];
        }
        w += mx;
        sm += 64 * mx;
    }
    *wave = w;
    *smooth = sm;
}

// The faces of a cell may be summed in any order (Eq. 3's face sum), so per
// half-warp each cell's faces are permuted among its slots by a local search
// (best permutation per cell in turn, from the caller's order and from random
// ones, keeping the fewest wavefronts).  perm[c * mf + j] = the face (old slot)
// that slot j of cell c takes.  Returns {wavefronts before, after}.
inline std::pair<int64_t, int64_t> order_face_slots(std::vector<uint16_t> &sidx, int32_t nc, int mf,
                                                    std::vector<uint8_t> &perm) {
    perm.assign((size_t)nc * mf, 0);
    for (int32_t c = 0; c < nc; ++c)
        for (int j = 0; j < mf; ++j) perm[(size_t)c * mf + j] = (uint8_t)j;
    if (mf > 8) return {0, 0};
    std::vector<std::array<uint8_t, 8>> perms;  // candidate permutations of a cell's slots
    {
        std::array<uint8_t, 8> p{};
        for (int j = 0; j < mf; ++j) p[j] = (uint8_t)j;
        if (mf <= 4) {
            do perms.push_back(p); while (std::next_permutation(p.begin(), p.begin() + mf));
        } else {
            perms.push_back(p);
            for (int a = 0; a < mf; ++a)
                for (int b = a + 1; b < mf; ++b) {
                    auto q = p;
                    std::swap(q[a], q[b]);
                    perms.push_back(q);
                }
        }
    }
    const int restarts = nc <= (1 << 18) ? 4 : 1;
    uint64_t rng = 0x9e3779b97f4a7c15ull;  // (deterministic)
    auto next = [&rng]() {
        rng ^= rng << 13;
        rng ^= rng >> 7;
        rng ^= rng << 17;
        return rng;
    };
    int64_t before = 0, after = 0;
    uint16_t orig[16][8], col[8][16], best_col[8][16];
    uint8_t cur_p[16][8], best_p[16][8];
    for (int32_t h0 = 0; h0 < nc; h0 += 16) {
        const int n = std::min<int32_t>(16, nc - h0);
        for (int l = 0; l < n; ++l)
            for (int j = 0; j < mf; ++j) {
                orig[l][j] = sidx[(size_t)j * nc + h0 + l];
                col[j][l] = orig[l][j];
                cur_p[l][j] = (uint8_t)j;
            }
        int wave, smooth;
        half_costs(col, mf, n, &wave, &smooth);
        before += wave;
        int best_wave = wave;
        std::memcpy(best_col, col, sizeof(col));
        std::memcpy(best_p, cur_p, sizeof(cur_p));
        for (int r = 0; r < restarts; ++r) {
            for (int l = 0; l < n; ++l) {  // start: the caller's order, then random ones
                const auto &p = perms[r == 0 ? 0 : next() % perms.size()];
                for (int j = 0; j < mf; ++j) {
                    cur_p[l][j] = p[j];
                    col[j][l] = orig[l][p[j]];
                }
            }
            half_costs(col, mf, n, &wave, &smooth);
            for (int pass = 0; pass < 6; ++pass) {
                bool improved = false;
                for (int l = 0; l < n; ++l) {
                    int bs = smooth, bw = wave, bi = -1;
                    for (size_t pi = 0; pi < perms.size(); ++pi) {
                        for (int j = 0; j < mf; ++j) col[j][l] = orig[l][perms[pi][j]];
                        int w2, s2;
                        half_costs(col, mf, n, &w2, &s2);
                        if (s2 < bs) bs = s2, bw = w2, bi = (int)pi;
                    }
                    const uint8_t *p = bi >= 0 ? perms[bi].data() : cur_p[l];
                    uint8_t keep[8];
                    for (int j = 0; j < mf; ++j) keep[j] = p[j];
                    for (int j = 0; j < mf; ++j) {
                        cur_p[l][j] = keep[j];
                        col[j][l] = orig[l][keep[j]];
                    }
                    if (bi >= 0) {
                        smooth = bs;
                        wave = bw;
                        improved = true;
                    }
                }
                if (!improved) break;
            }
            if (wave < best_wave) {
                best_wave = wave;
                std::memcpy(best_col, col, sizeof(col));
                std::memcpy(best_p, cur_p, sizeof(cur_p));
            }
        }
        after += best_wave;
        for (int l = 0; l < n; ++l)
            for (int j = 0; j < mf; ++j) {
                sidx[(size_t)j * nc + h0 + l] = best_col[j][l];
                perm[(size_t)(h0 + l) * mf + j] = best_p[l][j];
            }
    }
    return {before, after};
}

// Positions of a tile's staged values (halo cells, then ghosts; item k is read
// by the half-warps readers[k], deg[H][k] counts the in-tile upwind reads of
// half-warp H in bank class k): the most-read values first, each at the free
// position of [base, base + cap) whose bank class adds least to the class
// counts of the half-warps that read it.  pos[k] = the position of item k.
inline void place_staged(const std::vector<std::vector<int32_t>> &readers, int deg[][16], int32_t base, int32_t cap,
                         std::vector<int32_t> &pos) {
    const int32_t n = (int32_t)readers.size();
    std::vector<int32_t> order(n), freep(cap);
    for (int32_t k = 0; k < n; ++k) order[k] = k;
    std::stable_sort(order.begin(), order.end(),
                     [&](int32_t a, int32_t b) { return readers[a].size() > readers[b].size(); });
    for (int32_t p = 0; p < cap; ++p) freep[p] = base + p;
    pos.assign(n, -1);
    for (const int32_t k : order) {
        size_t bi = 0;
        int bs = INT_MAX;
        for (size_t fi = 0; fi < freep.size(); ++fi) {
            int sc = 0;
            for (const int32_t H : readers[k]) sc += 2 * deg[H][freep[fi] & 15] + 1;
            if (sc < bs) bs = sc, bi = fi;
        }
        const int32_t p = freep[bi];
        freep.erase(freep.begin() + (std::ptrdiff_t)bi);
        for (const int32_t H : readers[k]) ++deg[H][p & 15];
        pos[k] = p;
    }
}

}  // namespace bte_host
