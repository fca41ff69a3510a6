// bte_layout.cu -- structure detection for bte_create (see bte_internal.h):
// the structured 2-D / 3-D grids the box kernel takes (lattice walk from the
// corner cell, uniform A / V per axis, side kinds, orbit tables), the tensor
// maps of its bulk copies, z-slab cell partitions of box grids, and the owned
// mesh + halo plan of a cell partition.
#include "bte_internal.h"

#include <map>
#include <set>

namespace bte_host {


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

}  // namespace bte_host
