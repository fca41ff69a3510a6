"""Seeded synthetic inputs for the phonon-BTE explicit step.

This module is the ONE thing the CUDA path and the CPU oracle share.  It
produces plain arrays (meshes, band tables, direction sets, boundary
conditions, initial-condition multipliers, time steps) and holds none of the
method's arithmetic: no flux, no relaxation, no equilibrium intensity, no
temperature relation.  Each side turns these arrays into the method itself.

Shapes of the paper's workloads (citations are /root/reference/PAPER.md lines):
  * FVM mesh of polygonal/polyhedral cells with m faces, face areas A_i,
    outward normals and CELL1/CELL2 adjacency (Eq. 3; L719-722).
    Generated here as uniform Cartesian quads/hexes stored face by face.
  * 40 spectral bands -> 40 LA + 15 TA = 55 band-rows (L105-108, L507-514,
    L593-594; Appendix).  External Si dispersion: SURVEY 8(c) #13.
  * 2-D: 20 uniformly distributed directions (L594-596); 3-D: 20 x 20 = 400
    (L514-516).  SURVEY 8(c) #15 gives the midpoint sets used here.
  * Fig. 1 scenario: cold isothermal wall at 300, opposite isothermal wall with a
    centred Gaussian hot spot (peak 350, 1/e^2 distance 10 um), symmetric sides,
    IC = equilibrium at 300, 525 um square, 120 x 120 (L578-600, L617-623).

Every random draw uses numpy.random.default_rng with an explicit seed.
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field

import numpy as np

# Wall codes of a Cartesian mesh, in per-cell face-slot order.
WALL_XM, WALL_XP, WALL_YM, WALL_YP, WALL_ZM, WALL_ZP = range(6)
ISOTHERMAL, SYMMETRY = 0, 1
LA, TA = 0, 1

SEED = 2024


# --------------------------------------------------------------------------- mesh
def gen_mesh(shape, spacing):
    """Uniform Cartesian mesh stored as a face-based FVM mesh.

    shape = (nx, ny) or (nx, ny, nz); spacing = (dx, dy[, dz]) in metres.
    2-D meshes are 3-D with unit depth and n_z = 0 (A = edge
    length x 1, V = cell area).  Cell id c = i + nx*(j + ny*k).  Faces of each
    cell are stored in slot order -x, +x, -y, +y[, -z, +z]; face_nbr >= 0 is the
    neighbour cell, face_nbr < 0 encodes boundary face id = -1 - face_nbr,
    numbered in storage order.
    """
    shape = tuple(int(s) for s in shape)
    spacing = tuple(float(h) for h in spacing)
    dim = len(shape)
    assert dim in (2, 3) and len(spacing) == dim
    nx, ny = shape[0], shape[1]
    nz = shape[2] if dim == 3 else 1
    dx, dy = spacing[0], spacing[1]
    dz = spacing[2] if dim == 3 else 1.0
    nc = nx * ny * nz
    mf = 2 * dim
    c = np.arange(nc, dtype=np.int64)
    i = c % nx
    j = (c // nx) % ny
    k = c // (nx * ny)
    nbr = np.empty((nc, mf), dtype=np.int64)
    area = np.empty((nc, mf), dtype=np.float64)
    normal = np.zeros((nc, mf, 3), dtype=np.float64)
    wall = np.full((nc, mf), -1, dtype=np.int64)
    specs = [  # (axis, sign, index array, extent, stride, area)
        (0, -1, i, nx, 1, dy * dz), (0, +1, i, nx, 1, dy * dz),
        (1, -1, j, ny, nx, dx * dz), (1, +1, j, ny, nx, dx * dz),
    ]
    if dim == 3:
        specs += [(2, -1, k, nz, nx * ny, dx * dy), (2, +1, k, nz, nx * ny, dx * dy)]
    for slot, (axis, sign, idx, ext, stride, a) in enumerate(specs):
        inside = (idx > 0) if sign < 0 else (idx < ext - 1)
        nbr[:, slot] = np.where(inside, c + sign * stride, -1)
        wall[:, slot] = np.where(inside, -1, slot)
        area[:, slot] = a
        normal[:, slot, axis] = float(sign)
    bmask = nbr < 0
    bid = np.cumsum(bmask.ravel()) - 1
    flat_nbr = nbr.ravel().copy()
    flat_nbr[bmask.ravel()] = -1 - bid[bmask.ravel()]
    centre = np.stack([(i + 0.5) * dx, (j + 0.5) * dy, (k + 0.5) * dz], axis=1)
    half = np.zeros((mf, 3))
    for slot, (axis, sign, *_rest) in enumerate(specs):
        half[slot, axis] = sign * 0.5 * (dx, dy, dz)[axis]
    fcent = centre[:, None, :] + half[None, :, :]
    bface_centre = fcent.reshape(-1, 3)[bmask.ravel()]
    bface_wall = wall.ravel()[bmask.ravel()]
    return {
        "dim": dim,
        "n_cells": nc,
        "face_offsets": np.arange(0, nc * mf + 1, mf, dtype=np.int64),
        "face_nbr": flat_nbr,
        "face_area": area.ravel(),
        "face_normal": normal.reshape(-1, 3),
        "cell_volume": np.full(nc, dx * dy * dz),
        # metadata (not part of the method's input)
        "shape": shape,
        "spacing": spacing if dim == 3 else (dx, dy),
        "cell_centre": centre,
        "bface_centre": bface_centre,
        "bface_wall": bface_wall,
        "n_bfaces": int(bmask.sum()),
    }


def gen_mesh_tri(shape, spacing, seed=SEED):
    """Unstructured 2-D triangle mesh: the nx x ny quad grid
    with every quad split along a seeded random diagonal, stored face-based
    like gen_mesh (3 faces per cell, unit depth, outward unit normals, boundary
    faces on the rectangle's sides with the same wall codes).  Cell 2 q is the
    triangle holding the quad's bottom edge, 2 q + 1 the one holding its top
    edge (q = i + nx j)."""
    nx, ny = (int(v) for v in shape)
    dx, dy = (float(h) for h in spacing)
    rng = np.random.default_rng([seed, 7])
    diag = rng.integers(0, 2, size=(ny, nx))  # 0: v00-v11, 1: v10-v01
    dl = math.hypot(dx, dy)
    cid = lambda i, j, t: 2 * (i + nx * j) + t
    off, nbr, area, nrm, cen = [0], [], [], [], []
    bcent, bwall = [], []

    def owner_left(i, j):   # triangle of quad (i, j) holding its left edge
        return cid(i, j, 1 if diag[j, i] == 0 else 0)

    def owner_right(i, j):
        return cid(i, j, 0 if diag[j, i] == 0 else 1)

    for j in range(ny):
        for i in range(nx):
            x0, y0 = i * dx, j * dy
            v00, v10, v01, v11 = (x0, y0), (x0 + dx, y0), (x0, y0 + dy), (x0 + dx, y0 + dy)
            d = diag[j, i]
            for t in (0, 1):
                faces = []  # (neighbour or ('wall', code), area, normal, face centre)
                if t == 0:  # holds the bottom edge
                    faces.append((cid(i, j - 1, 1) if j > 0 else ("w", WALL_YM), dx, (0.0, -1.0), (x0 + dx / 2, y0)))
                else:       # holds the top edge
                    faces.append((cid(i, j + 1, 0) if j < ny - 1 else ("w", WALL_YP), dx, (0.0, 1.0),
                                  (x0 + dx / 2, y0 + dy)))
                holds_left = (d == 0 and t == 1) or (d == 1 and t == 0)
                if holds_left:
                    faces.append((owner_right(i - 1, j) if i > 0 else ("w", WALL_XM), dy, (-1.0, 0.0),
                                  (x0, y0 + dy / 2)))
                else:
                    faces.append((owner_left(i + 1, j) if i < nx - 1 else ("w", WALL_XP), dy, (1.0, 0.0),
                                  (x0 + dx, y0 + dy / 2)))
                if d == 0:  # diagonal v00 - v11: lower-right triangle's outward normal points up-left
                    n = (-dy / dl, dx / dl) if t == 0 else (dy / dl, -dx / dl)
                else:       # diagonal v10 - v01: lower-left triangle's outward normal points up-right
                    n = (dy / dl, dx / dl) if t == 0 else (-dy / dl, -dx / dl)
                faces.append((cid(i, j, 1 - t), dl, n, (x0 + dx / 2, y0 + dy / 2)))
                verts = {(0, 0): (v00, v10, v11), (0, 1): (v00, v11, v01),
                         (1, 0): (v00, v10, v01), (1, 1): (v10, v11, v01)}[(d, t)]
                cen.append((sum(v[0] for v in verts) / 3, sum(v[1] for v in verts) / 3, 0.5))
                for nb, a, nn, fc in faces:
                    if isinstance(nb, tuple):
                        bwall.append(nb[1])
                        bcent.append((fc[0], fc[1], 0.5))
                        nbr.append(-len(bwall))
                    else:
                        nbr.append(nb)
                    area.append(a)
                    nrm.append((nn[0], nn[1], 0.0))
                off.append(len(nbr))
    nc = 2 * nx * ny
    return {
        "dim": 2, "n_cells": nc,
        "face_offsets": np.asarray(off, np.int64), "face_nbr": np.asarray(nbr, np.int64),
        "face_area": np.asarray(area, np.float64), "face_normal": np.asarray(nrm, np.float64),
        "cell_volume": np.full(nc, 0.5 * dx * dy),
        "shape": (nx, ny), "spacing": (dx, dy), "cell_centre": np.asarray(cen, np.float64),
        "bface_centre": np.asarray(bcent, np.float64), "bface_wall": np.asarray(bwall, np.int64),
        "n_bfaces": len(bwall), "triangles": True,
    }


def general_dt_bound(mesh, bands, dirs, t_max=None):
    """Positivity bound on any face-based mesh: 1 / max_b (1/tau_b + v_b S),
    S = max_{c,d} sum_f (A_f / V_c) max(s_d . n_f, 0) (used to pick
    dt for the synthetic configs, as cartesian_dt_bound on Cartesian grids)."""
    off = mesh["face_offsets"]
    owner = np.repeat(np.arange(mesh["n_cells"]), np.diff(off))
    g = (mesh["face_area"] / mesh["cell_volume"][owner])[:, None] * mesh["face_normal"]
    mu = np.maximum(g @ dirs["s"].T, 0.0)  # [faces][dirs]
    per_cell = np.zeros((mesh["n_cells"], dirs["n_dirs"]))
    np.add.at(per_cell, owner, mu)
    smax = float(per_cell.max())
    if bands.get("rate_a") is not None:
        t = 350.0 if t_max is None else float(t_max)
        inv_tau = bands["rate_a"] + bands["rate_b"] * t * np.exp(-bands["rate_theta"] / t)
    else:
        inv_tau = np.where(np.isinf(bands["tau"]), 0.0, 1.0 / bands["tau"])
    return 1.0 / float(np.max(inv_tau + bands["vg"] * smax))


def permute_mesh(mesh, seed=SEED):
    """Random relabelling of cells and of each cell's face order (pin P11).

    Returns (mesh', perm) with new cell id n holding old cell perm[n].  Boundary
    face ids keep their numbering so BC arrays stay valid.
    """
    rng = np.random.default_rng(seed)
    nc = mesh["n_cells"]
    perm = rng.permutation(nc)
    inv = np.empty(nc, dtype=np.int64)
    inv[perm] = np.arange(nc)
    off = mesh["face_offsets"]
    nbr_out, area_out, nrm_out, off_out = [], [], [], [0]
    for new_c in range(nc):
        old_c = perm[new_c]
        lo, hi = off[old_c], off[old_c + 1]
        order = lo + rng.permutation(hi - lo)
        nb = mesh["face_nbr"][order].copy()
        inside = nb >= 0
        nb[inside] = inv[nb[inside]]
        nbr_out.append(nb)
        area_out.append(mesh["face_area"][order])
        nrm_out.append(mesh["face_normal"][order])
        off_out.append(off_out[-1] + (hi - lo))
    out = dict(mesh)
    out.update(
        face_offsets=np.asarray(off_out, dtype=np.int64),
        face_nbr=np.concatenate(nbr_out),
        face_area=np.concatenate(area_out),
        face_normal=np.concatenate(nrm_out),
        cell_volume=mesh["cell_volume"][perm],
        cell_centre=mesh["cell_centre"][perm],
    )
    return out, perm


def split_faces(mesh, every=3):
    """Split the first face of every `every`-th cell into two half-area faces
    with the same normal and neighbour (a hanging-node style polygon): such
    cells no longer have opposite-face pairs, which exercises the generic
    face-slot path.  Boundary faces are not split (ids stay unique)."""
    off, nbr = mesh["face_offsets"], mesh["face_nbr"]
    area, nrm = mesh["face_area"], mesh["face_normal"]
    o_off, o_nbr, o_area, o_nrm = [0], [], [], []
    for c in range(mesh["n_cells"]):
        lo, hi = off[c], off[c + 1]
        for f in range(lo, hi):
            if f == lo and c % every == 0 and nbr[f] >= 0:
                o_nbr += [nbr[f], nbr[f]]
                o_area += [0.5 * area[f], 0.5 * area[f]]
                o_nrm += [nrm[f], nrm[f]]
            else:
                o_nbr.append(nbr[f])
                o_area.append(area[f])
                o_nrm.append(nrm[f])
        o_off.append(len(o_nbr))
    out = dict(mesh)
    out.update(face_offsets=np.asarray(o_off, np.int64), face_nbr=np.asarray(o_nbr, np.int64),
               face_area=np.asarray(o_area), face_normal=np.asarray(o_nrm).reshape(-1, 3))
    return out


# --------------------------------------------------------------------------- bands
# External Si quadratic dispersion omega = v_s k + c k^2.
SI_LATTICE = 5.431e-10
SI_DISP = {LA: (9.01e3, -2.0e-7), TA: (5.23e3, -2.26e-7)}
TAU_A, TAU_B, TAU_THETA, TAU_TREF = 1.32e-45, 1.73e-19, 137.3, 300.0
HBAR = 1.054571817e-34  # only used for the band prefactor C_b below


def _omega_max(pol):
    v, cq = SI_DISP[pol]
    kmax = 2.0 * math.pi / SI_LATTICE
    return v * kmax + cq * kmax * kmax


def gen_bands_si(n_spectral):
    """Band-rows for n_spectral uniform bands over the LA branch.

    LA rows for every spectral band, then a TA row for every band whose upper
    edge lies below omega_max,TA (15 for N = 40, L105-107).  Per row: centre
    omega, width d_omega, group velocity v = v_s + 2 c k, a placeholder
    relaxation time and the intensity prefactor
    C_b = hbar omega k^2 d_omega / (8 pi^3) (external).
    """
    wmax_la, wmax_ta = _omega_max(LA), _omega_max(TA)
    dw = wmax_la / n_spectral
    rows = []
    for pol in (LA, TA):
        v, cq = SI_DISP[pol]
        for i in range(n_spectral):
            if pol == TA and (i + 1) * dw > wmax_ta:
                continue
            w = (i + 0.5) * dw
            k = 2.0 * w / (v + math.sqrt(v * v + 4.0 * cq * w))
            vg = v + 2.0 * cq * k
            rate = TAU_A * w ** 4 + TAU_B * w * w * TAU_TREF * math.exp(-TAU_THETA / TAU_TREF)
            pref = HBAR * w * k * k * dw / (8.0 * math.pi ** 3)
            rows.append((w, dw, vg, 1.0 / rate, pol, pref))
    a = np.array(rows, dtype=np.float64)
    return {
        "n_bands": len(rows),
        "omega": a[:, 0].copy(),
        "d_omega": a[:, 1].copy(),
        "vg": a[:, 2].copy(),
        "tau": a[:, 3].copy(),
        "polarization": a[:, 4].astype(np.int32),
        "C": a[:, 5].copy(),
        "n_spectral": n_spectral,
    }


def gen_bands_custom(omega, vg, tau, C, polarization=None, d_omega=None):
    """Explicit band table (used by the pins: gray, ballistic, 3-row sets)."""
    omega = np.atleast_1d(np.asarray(omega, dtype=np.float64))
    nb = omega.size
    bc = lambda x: np.broadcast_to(np.asarray(x, dtype=np.float64), (nb,)).copy()
    return {
        "n_bands": nb,
        "omega": omega.copy(),
        "d_omega": bc(d_omega if d_omega is not None else 1.0),
        "vg": bc(vg),
        "tau": bc(tau),
        "polarization": (np.zeros(nb, np.int32) if polarization is None
                         else np.asarray(polarization, np.int32)),
        "C": bc(C),
        "n_spectral": nb,
    }


def with_rate_law(bands, a=TAU_A, b=TAU_B, theta=TAU_THETA):
    """Temperature-dependent relaxation times: the same
    placeholder law as gen_bands_si's constant tau, kept as a function of the
    cell temperature, 1/tau_b(T) = a w^4 + b w^2 T exp(-theta/T), i.e. per row
    rate_a = a w^4, rate_b = b w^2, rate_theta = theta (external, Si-like)."""
    w = np.asarray(bands["omega"], dtype=np.float64)
    out = dict(bands)
    out["rate_a"] = a * w ** 4
    out["rate_b"] = b * w ** 2
    out["rate_theta"] = np.full(w.size, float(theta))
    return out


def select_bands(bands, rows):
    rows = np.asarray(rows)
    out = dict(bands)
    keys = ["omega", "d_omega", "vg", "tau", "polarization", "C"]
    keys += [k for k in ("rate_a", "rate_b", "rate_theta") if bands.get(k) is not None]
    for key in keys:
        out[key] = bands[key][rows].copy()
    out["n_bands"] = int(rows.size)
    return out


# --------------------------------------------------------------------------- directions
def gen_dirs_inplane(nd):
    """phi_j = (j + 1/2) 2 pi / nd in the x-y plane, w = 4 pi / nd."""
    phi = (np.arange(nd) + 0.5) * 2.0 * np.pi / nd
    s = np.stack([np.cos(phi), np.sin(phi), np.zeros(nd)], axis=1)
    return {"n_dirs": nd, "s": s, "w": np.full(nd, 4.0 * np.pi / nd)}


def gen_dirs_product(ntheta, nphi):
    """Midpoint polar x azimuthal set; w_ij = (cos th- - cos th+) dphi, sum 4 pi."""
    te = np.linspace(0.0, np.pi, ntheta + 1)
    th = 0.5 * (te[:-1] + te[1:])
    dphi = 2.0 * np.pi / nphi
    phi = (np.arange(nphi) + 0.5) * dphi
    T, P = np.meshgrid(th, phi, indexing="ij")
    s = np.stack([np.sin(T) * np.cos(P), np.sin(T) * np.sin(P), np.cos(T)], axis=-1).reshape(-1, 3)
    wt = (np.cos(te[:-1]) - np.cos(te[1:]))[:, None] * np.full((1, nphi), dphi)
    return {"n_dirs": ntheta * nphi, "s": s, "w": wt.reshape(-1)}


def gen_dirs_axes2d():
    """{+x, -x, +y, -y} with equal weights pi (pin P6)."""
    s = np.array([[1, 0, 0], [-1, 0, 0], [0, 1, 0], [0, -1, 0]], dtype=np.float64)
    return {"n_dirs": 4, "s": s, "w": np.full(4, np.pi)}


# --------------------------------------------------------------------------- BCs
def gen_bcs_walls(mesh, walls):
    """walls: {wall_code: (kind, t_wall or callable(face_centres)->t)}."""
    nbf = mesh["n_bfaces"]
    kind = np.full(nbf, -1, dtype=np.int32)
    t = np.zeros(nbf, dtype=np.float64)
    for code, (k, tw) in walls.items():
        sel = mesh["bface_wall"] == code
        kind[sel] = k
        if callable(tw):
            t[sel] = tw(mesh["bface_centre"][sel])
        else:
            t[sel] = float(tw)
    assert (kind >= 0).all(), "every boundary face needs a BC"
    return {"n_bfaces": nbf, "kind": kind, "t_wall": t}


def gen_bcs_uniform(mesh, kind, t_wall=300.0):
    nbf = mesh["n_bfaces"]
    return {"n_bfaces": nbf, "kind": np.full(nbf, kind, np.int32),
            "t_wall": np.full(nbf, float(t_wall))}


def gen_bcs_fig1(mesh, t_cold=300.0, t_hot=350.0, radius=10e-6, centre=None):
    """Fig. 1 (L578-600, L617-621).

    2-D: y = L_y isothermal with T_w = t_cold + (t_hot - t_cold) exp(-2 r^2/R^2)
    (R = 1/e^2 radius), y = 0 isothermal t_cold, x = 0 and x = L_x symmetric.
    3-D: the same on z (radial Gaussian in x-y), four sides symmetric.
    """
    dim = mesh["dim"]
    sh, hs = mesh["shape"], mesh["spacing"]
    lx, ly = sh[0] * hs[0], sh[1] * hs[1]
    if centre is None:
        centre = (0.5 * lx, 0.5 * ly)

    def hot(fc):
        if dim == 2:
            r2 = (fc[:, 0] - centre[0]) ** 2
        else:
            r2 = (fc[:, 0] - centre[0]) ** 2 + (fc[:, 1] - centre[1]) ** 2
        return t_cold + (t_hot - t_cold) * np.exp(-2.0 * r2 / radius ** 2)

    if dim == 2:
        walls = {WALL_XM: (SYMMETRY, 0.0), WALL_XP: (SYMMETRY, 0.0),
                 WALL_YM: (ISOTHERMAL, t_cold), WALL_YP: (ISOTHERMAL, hot)}
    else:
        walls = {WALL_XM: (SYMMETRY, 0.0), WALL_XP: (SYMMETRY, 0.0),
                 WALL_YM: (SYMMETRY, 0.0), WALL_YP: (SYMMETRY, 0.0),
                 WALL_ZM: (ISOTHERMAL, t_cold), WALL_ZP: (ISOTHERMAL, hot)}
    return gen_bcs_walls(mesh, walls)


# --------------------------------------------------------------------------- IC, dt
def ic_multiplier(nd, nc, band, eps, seed=SEED):
    """Seeded IC perturbation factor (1 + eps U(-1,1)) for one band-row, [nd][nc].

    Drawn per band-row so that large configs can be generated one slab at a
    time; the equilibrium value it multiplies is computed by each side.
    """
    if eps == 0.0:
        return np.ones((nd, nc))
    rng = np.random.default_rng([seed, int(band)])
    return 1.0 + eps * rng.uniform(-1.0, 1.0, size=(nd, nc))


def cartesian_dt_bound(mesh, bands, dirs, t_max=None):
    """Positivity bound of the explicit step on a uniform Cartesian mesh.

    1 / max_b (1/tau_b + v_b S), S = max_d sum_axis |s_axis| / h_axis (one face
    per axis is outgoing; A/V = 1/h).  Only used to choose dt for the synthetic
    configs ("dt = 0.5 x positivity bound").  With a rate law
    (with_rate_law) the rates are taken at t_max (default 350 K, the hot wall).
    """
    h = np.asarray(mesh["spacing"], dtype=np.float64)
    s = np.abs(dirs["s"][:, : mesh["dim"]])
    smax = float(np.max(np.sum(s / h[None, :], axis=1)))
    if bands.get("rate_a") is not None:
        t = 350.0 if t_max is None else float(t_max)
        inv_tau = bands["rate_a"] + bands["rate_b"] * t * np.exp(-bands["rate_theta"] / t)
        return 1.0 / float(np.max(inv_tau + bands["vg"] * smax))
    inv_tau = np.where(np.isinf(bands["tau"]), 0.0, 1.0 / bands["tau"])
    return 1.0 / float(np.max(inv_tau + bands["vg"] * smax))


# --------------------------------------------------------------------------- configs
@dataclass
class Config:
    name: str
    mesh: dict
    bands: dict
    dirs: dict
    bcs: dict
    t_init: float
    dt: float
    nsteps: int
    ic_eps: float = 0.0
    temp_rule: int = 0
    note: str = ""
    extra: dict = field(default_factory=dict)
    ic_mult: object = None  # callable (nd, nc, band) -> [nd][nc] IC multiplier (instead of ic_eps)

    @property
    def n_updates_per_step(self):
        return self.mesh["n_cells"] * self.dirs["n_dirs"] * self.bands["n_bands"]


def make_config(name, variant="scaled"):
    """BASELINE.json configs C1-C5 as exact arrays.

    variant "scaled": seeded IC perturbation and dt = 0.5 x positivity bound
    (parity/bench); "paper": C3 exactly as the paper (IC 300 K, dt = 1 ps).
    """
    if name == "C1":
        mesh = gen_mesh((16, 16), (1e-6, 1e-6))
        bands = gen_bands_si(1)
        dirs = gen_dirs_inplane(8)
        bcs = gen_bcs_fig1(mesh, radius=2e-6)
        nsteps, eps = 50, 0.05
    elif name == "C2":
        mesh = gen_mesh((64, 64), (1e-6, 1e-6))
        bands = gen_bands_si(10)
        dirs = gen_dirs_product(4, 20)
        bcs = gen_bcs_fig1(mesh, radius=4e-6)
        nsteps, eps = 500, 0.10
    elif name in ("C3", "C3t"):
        # C3t: the same domain as an unstructured triangle mesh
        # (every quad split on a seeded diagonal: 28,800 cells) for the generic-face path
        h = 525e-6 / 120
        mesh = gen_mesh((120, 120), (h, h)) if name == "C3" else gen_mesh_tri((120, 120), (h, h))
        bands = gen_bands_si(40)
        dirs = gen_dirs_product(20, 20)
        bcs = gen_bcs_fig1(mesh, radius=10e-6)
        nsteps, eps = 1000, 0.10
    elif name in ("C4", "C5"):
        n = (64, 64, 32) if name == "C4" else (96, 96, 96)
        h = 8.2e-6
        mesh = gen_mesh(n, (h, h, h))
        bands = gen_bands_si(40)
        dirs = gen_dirs_product(20, 20)
        bcs = gen_bcs_fig1(mesh, radius=4 * h)
        nsteps, eps = (100, 0.10) if name == "C4" else (20, 0.10)
    elif name in ("C6", "C6t"):
        # Fig. 10 (L1169-1178): a smaller, elongated material,
        # heat source in one corner, specular left/right, isothermal bottom;
        # colour scale 100-150 K.  Reading: 40 x 160 um (1:4), the top wall
        # isothermal 100 K with a 150 K Gaussian (1/e^2 radius 10 um) centred on
        # the top-left corner, bottom 100 K, IC 100 K; 10 spectral bands (13
        # rows), the paper's 2-D set of 20 directions (L594-595).  C6t: the same
        # domain as an unstructured triangle mesh (each quad split on a seeded
        # random diagonal).
        shape, h = (20, 80), 2e-6
        mesh = gen_mesh(shape, (h, h)) if name == "C6" else gen_mesh_tri(shape, (h, h))
        bands = gen_bands_si(10)
        dirs = gen_dirs_inplane(20)
        bcs = gen_bcs_fig1(mesh, t_cold=100.0, t_hot=150.0, radius=10e-6, centre=(0.0, shape[1] * h))
        nsteps, eps = 200, 0.10
    else:
        raise ValueError(f"unknown config {name}")
    t_init = 100.0 if name in ("C6", "C6t") else 300.0
    bound = general_dt_bound(mesh, bands, dirs) if mesh.get("triangles") else cartesian_dt_bound(mesh, bands, dirs)
    if variant == "paper":
        assert name in ("C3", "C6", "C6t")
        dt, eps = (1e-12 if name == "C3" else 0.5 * bound), 0.0
    else:
        dt = 0.5 * bound
    return Config(name=name, mesh=mesh, bands=bands, dirs=dirs, bcs=bcs, t_init=t_init,
                  dt=dt, nsteps=nsteps, ic_eps=eps, extra={"dt_bound": bound})


def small_3d_config(shape=(6, 5, 4), n_spectral=2, ntheta=4, nphi=8, eps=0.1, h=1e-6):
    """Tiny 3-D Fig.-1-style problem (parity on several tiles + ragged tails)."""
    mesh = gen_mesh(shape, (h, h, h))
    bands = gen_bands_si(n_spectral)
    dirs = gen_dirs_product(ntheta, nphi)
    bcs = gen_bcs_fig1(mesh, radius=2 * h)
    bound = cartesian_dt_bound(mesh, bands, dirs)
    return Config(name=f"3d{shape}", mesh=mesh, bands=bands, dirs=dirs, bcs=bcs,
                  t_init=300.0, dt=0.5 * bound, nsteps=10, ic_eps=eps, extra={"dt_bound": bound})


# --------------------------------------------------------------------------- ENOCONV case
def failing_strip_config(amp=11.0, comp=9.5, nx=12, x0=1):
    """A state whose temperature solve fails in step 4 (BTE_ENOCONV semantics,
    SURVEY 8(b)): a 2-D nx x 2 strip (1 um cells), isothermal 300 K ends,
    specular top / bottom, the 4 diagonal in-plane directions, two gray-like
    rows without scattering (tau = inf, temperature rule R1) whose group
    velocities differ by 2x.  At cells x = 1, 2 the +x directions of row 0 are
    set to -amp x equilibrium and those of row 1 to (1 + comp) x equilibrium
    (cells x0, x0 + 1 in general):
    the energy starts positive, but the fast negative row-0 pulse outruns the
    slow compensating row-1 pulse and a cell's energy turns negative after a
    few steps (step 4 for the defaults, found with the oracle).  dt = the
    positivity bound.  Multipliers only; each side evaluates its own I0."""
    h = 1e-6
    mesh = gen_mesh((nx, 2), (h, h))
    bands = gen_bands_custom(omega=[2e13, 3e13], vg=[6000.0, 3000.0], tau=np.inf, C=[1e9, 1e9])
    dirs = gen_dirs_inplane(4)
    bcs = gen_bcs_walls(mesh, {WALL_XM: (ISOTHERMAL, 300.0), WALL_XP: (ISOTHERMAL, 300.0),
                               WALL_YM: (SYMMETRY, 0.0), WALL_YP: (SYMMETRY, 0.0)})
    dp = np.where(dirs["s"][:, 0] > 0)[0]
    cells = np.array([y * nx + x for y in range(2) for x in (x0, x0 + 1)])

    def mult(nd, nc, band):
        m = np.ones((nd, nc))
        m[np.ix_(dp, cells)] = -amp if band == 0 else 1.0 + comp
        return m

    return Config(name="fail-strip", mesh=mesh, bands=bands, dirs=dirs, bcs=bcs, t_init=300.0,
                  dt=cartesian_dt_bound(mesh, bands, dirs), nsteps=10, temp_rule=1, ic_mult=mult,
                  note="temperature solve fails in step 4")
