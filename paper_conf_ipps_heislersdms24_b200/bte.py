"""Thin ctypes binding of libbte.so (include/bte.h): argument marshalling only.

Every step of the method runs in the library's CUDA kernels; this module only
converts NumPy arrays / torch streams into the C structs and checks status
codes.  There is no fallback: if libbte.so is missing or cannot be loaded,
importing this module raises.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
# BTE_LIB selects an experiment build of the same library (tools/); default in-tree libbte.so
LIB_PATH = os.environ.get("BTE_LIB") or os.path.join(_HERE, "libbte.so")

BTE_OK, BTE_EINVAL, BTE_ENOMEM, BTE_ECUDA, BTE_ENCCL, BTE_ENOCONV, BTE_ESTATE = range(7)
BTE_FLAG_PROFILE = 1
BTE_FLAG_GENERIC_FACES = 2
BTE_FLAG_NO_TMA = 4
BTE_FLAG_NO_BOX = 16
ISOTHERMAL, SYMMETRY = 0, 1


class BTEError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"{_STATUS.get(status, status)}: {msg}")
        self.status = status


_STATUS = {0: "BTE_OK", 1: "BTE_EINVAL", 2: "BTE_ENOMEM", 3: "BTE_ECUDA", 4: "BTE_ENCCL",
           5: "BTE_ENOCONV", 6: "BTE_ESTATE"}


class Mesh(C.Structure):
    _fields_ = [("dim", C.c_int32), ("n_cells", C.c_int64), ("face_offsets", C.c_void_p),
                ("face_nbr", C.c_void_p), ("face_area", C.c_void_p), ("face_normal", C.c_void_p),
                ("cell_volume", C.c_void_p), ("cell_centre", C.c_void_p)]


class Bands(C.Structure):
    _fields_ = [("n_bands", C.c_int32), ("omega", C.c_void_p), ("d_omega", C.c_void_p),
                ("vg", C.c_void_p), ("tau", C.c_void_p), ("polarization", C.c_void_p),
                ("i0_prefactor", C.c_void_p), ("rate_a", C.c_void_p), ("rate_b", C.c_void_p),
                ("rate_theta", C.c_void_p)]


class Dirs(C.Structure):
    _fields_ = [("n_dirs", C.c_int32), ("s", C.c_void_p), ("w", C.c_void_p)]


class Bcs(C.Structure):
    _fields_ = [("n_bfaces", C.c_int64), ("kind", C.c_void_p), ("t_wall", C.c_void_p)]


class Options(C.Structure):
    _fields_ = [("t_init", C.c_double), ("temp_rule", C.c_int32), ("newton_rtol", C.c_double),
                ("newton_max_iter", C.c_int32), ("rank", C.c_int32), ("world", C.c_int32),
                ("device", C.c_int32), ("nccl_unique_id", C.c_void_p), ("stream", C.c_void_p),
                ("flags", C.c_uint32), ("max_spare_slabs", C.c_int32), ("block_threads", C.c_int32),
                ("band_group", C.c_int32), ("dir_chunk", C.c_int32), ("cell_part", C.c_void_p),
                ("n_cell_parts", C.c_int32), ("group", C.c_void_p), ("rates_now", C.c_int32)]


class Stats(C.Structure):
    _fields_ = [("steps", C.c_int64), ("kernel_launches", C.c_int64), ("updates", C.c_int64),
                ("ms_flux_interior", C.c_double), ("ms_flux_boundary", C.c_double),
                ("ms_allreduce", C.c_double), ("ms_newton", C.c_double), ("ms_total", C.c_double),
                ("newton_iter_max", C.c_int32), ("spare_slabs", C.c_int32),
                ("n_interior_cells", C.c_int32), ("band_group", C.c_int32),
                ("block_threads", C.c_int32), ("dir_chunks", C.c_int32), ("flux_variant", C.c_int32),
                ("ms_halo", C.c_double), ("halo_bytes", C.c_int64), ("flux_launches", C.c_int64),
                ("graph_replays", C.c_int64)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


FLUX_VARIANTS = {0: "generic", 3: "tma", 4: "tma-uniform", 6: "box", 7: "tma-generic"}

EXPORTS = ["bte_options_default", "bte_create", "bte_step", "bte_dt_bound", "bte_get_temperature",
           "bte_get_intensity", "bte_set_intensity", "bte_solve_temperature", "bte_set_equilibrium",
           "bte_band_range", "bte_step_begin", "bte_get_energy", "bte_set_energy", "bte_step_finish",
           "bte_get_stats", "bte_reset_stats", "bte_nccl_unique_id", "bte_last_error",
           "bte_status_string", "bte_destroy", "bte_get_temperature_rule", "bte_local_cells",
           "bte_halo_size", "bte_halo_export", "bte_halo_import", "bte_group_create", "bte_group_destroy"]


def _load():
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: build it with "
                          "`python -m paper_conf_ipps_heislersdms24_b200.build` (no CPU fallback exists)")
    if "BTE_NCCL_LIB" not in os.environ:
        try:
            import nvidia.nccl  # type: ignore
            cand = os.path.join(list(nvidia.nccl.__path__)[0], "lib", "libnccl.so.2")
            if os.path.exists(cand):
                os.environ["BTE_NCCL_LIB"] = cand
        except Exception:
            pass
    lib = C.CDLL(LIB_PATH)
    vp, i32, i64, dbl = C.c_void_p, C.c_int32, C.c_int64, C.c_double
    P = C.POINTER
    sig = {
        "bte_options_default": ([P(Options)], i32),
        "bte_create": ([P(Mesh), P(Bands), P(Dirs), P(Bcs), P(Options), P(vp)], i32),
        "bte_step": ([vp, dbl, i64], i32),
        "bte_dt_bound": ([vp, P(dbl)], i32),
        "bte_get_temperature": ([vp, vp], i32),
        "bte_get_temperature_rule": ([vp, i32, vp], i32),
        "bte_get_intensity": ([vp, i32, i32, vp], i32),
        "bte_set_intensity": ([vp, i32, i32, vp], i32),
        "bte_solve_temperature": ([vp], i32),
        "bte_set_equilibrium": ([vp, vp], i32),
        "bte_band_range": ([vp, P(i32), P(i32)], i32),
        "bte_step_begin": ([vp, dbl], i32),
        "bte_get_energy": ([vp, vp], i32),
        "bte_set_energy": ([vp, vp], i32),
        "bte_step_finish": ([vp], i32),
        "bte_get_stats": ([vp, P(Stats)], i32),
        "bte_reset_stats": ([vp], i32),
        "bte_nccl_unique_id": ([vp], i32),
        "bte_last_error": ([vp], C.c_char_p),
        "bte_status_string": ([i32], C.c_char_p),
        "bte_destroy": ([vp], None),
        "bte_local_cells": ([vp, P(i64), vp], i32),
        "bte_halo_size": ([vp, i32, P(i64), P(i64)], i32),
        "bte_halo_export": ([vp, i32, vp], i32),
        "bte_halo_import": ([vp, i32, vp], i32),
        "bte_group_create": ([i32, P(vp)], i32),
        "bte_group_destroy": ([vp], None),
    }
    for name, (args, res) in sig.items():
        fn = getattr(lib, name)
        fn.argtypes = args
        fn.restype = res
    return lib


lib = _load()


def _check(status, ctx=None):
    if status != BTE_OK:
        msg = lib.bte_last_error(ctx).decode()
        raise BTEError(status, msg)


def _p(a):
    return a.ctypes.data_as(C.c_void_p)


def nccl_unique_id() -> bytes:
    buf = C.create_string_buffer(128)
    _check(lib.bte_nccl_unique_id(C.cast(buf, C.c_void_p)))
    return buf.raw


class Group:
    """In-process communicator of `world` ranks (bte_group_create): every rank
    is a host thread of this process with its own Solver(group=...), calling
    the collective methods (step, solve_temperature, ...) from that thread.
    The library's per-step exchanges then run as device copies between the
    ranks (any device, several may share one).  Close it after the solvers."""

    def __init__(self, world):
        h = C.c_void_p()
        _check(lib.bte_group_create(int(world), C.byref(h)))
        self.handle, self.world = h, int(world)

    def close(self):
        if getattr(self, "handle", None):
            lib.bte_group_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()


class Solver:
    """One bte_ctx.  Arrays in caller cell order; I is [bands][dirs][cells].

    locality: pass the mesh's cell centroids (if the dict has them) as the
    library's internal-ordering hint; results are identical either way."""

    def __init__(self, mesh, bands, dirs, bcs, *, t_init=300.0, temp_rule=0, newton_rtol=1e-12,
                 newton_max_iter=50, rank=0, world=1, device=0, nccl_id: bytes | None = None,
                 stream=None, profile=False, max_spare_slabs=0, block_threads=0, band_group=0,
                 generic_faces=False, locality=True, dir_chunk=0, tma=True, box=True,
                 cell_part=None, n_cell_parts=1, group: Group | None = None, i0_prefactor=True,
                 rates_now=False):
        f64 = lambda x: np.ascontiguousarray(x, dtype=np.float64)
        i64 = lambda x: np.ascontiguousarray(x, dtype=np.int64)
        i32 = lambda x: np.ascontiguousarray(x, dtype=np.int32)
        k = self._keep = dict(
            off=i64(mesh["face_offsets"]), nbr=i64(mesh["face_nbr"]), area=f64(mesh["face_area"]),
            nrm=f64(mesh["face_normal"]), vol=f64(mesh["cell_volume"]),
            cen=f64(mesh["cell_centre"]) if (locality and mesh.get("cell_centre") is not None) else None,
            omega=f64(bands["omega"]), dw=f64(bands.get("d_omega", np.ones(bands["n_bands"]))),
            vg=f64(bands["vg"]), tau=f64(bands["tau"]),
            pol=i32(bands.get("polarization", np.zeros(bands["n_bands"]))), C=f64(bands["C"]),
            s=f64(dirs["s"]), w=f64(dirs["w"]), kind=i32(bcs["kind"]), tw=f64(bcs["t_wall"]),
        )
        law = bands.get("rate_a") is not None  # temperature-dependent relaxation times (N1)
        if law:
            k.update(ra=f64(bands["rate_a"]), rb=f64(bands["rate_b"]), rth=f64(bands["rate_theta"]))
        self.n_cells, self.n_bands, self.n_dirs = int(mesh["n_cells"]), int(bands["n_bands"]), int(dirs["n_dirs"])
        m = Mesh(int(mesh["dim"]), self.n_cells, _p(k["off"]).value, _p(k["nbr"]).value, _p(k["area"]).value,
                 _p(k["nrm"]).value, _p(k["vol"]).value, _p(k["cen"]).value if k["cen"] is not None else None)
        # i0_prefactor=False: pass NULL, the library derives C_b from its built-in dispersion
        b = Bands(self.n_bands, _p(k["omega"]).value, _p(k["dw"]).value, _p(k["vg"]).value, _p(k["tau"]).value,
                  _p(k["pol"]).value, _p(k["C"]).value if i0_prefactor else None,
                  _p(k["ra"]).value if law else None, _p(k["rb"]).value if law else None,
                  _p(k["rth"]).value if law else None)
        d = Dirs(self.n_dirs, _p(k["s"]).value, _p(k["w"]).value)
        bc = Bcs(int(bcs["n_bfaces"]), _p(k["kind"]).value, _p(k["tw"]).value)
        o = Options()
        _check(lib.bte_options_default(C.byref(o)))
        o.t_init, o.temp_rule, o.newton_rtol, o.newton_max_iter = float(t_init), int(temp_rule), float(newton_rtol), int(newton_max_iter)
        o.rank, o.world, o.device = int(rank), int(world), int(device)
        self._nccl_buf = None
        if nccl_id is not None:  # world > 1 and None: the caller reduces E (split-step calls)
            if len(nccl_id) != 128:
                raise ValueError("the NCCL id is 128 bytes (from nccl_unique_id() on rank 0)")
            self._nccl_buf = C.create_string_buffer(bytes(nccl_id), 128)
            o.nccl_unique_id = C.cast(self._nccl_buf, C.c_void_p).value
        if stream is not None:
            o.stream = int(getattr(stream, "cuda_stream", stream))
        if group is not None:
            self._group = group  # (kept alive while the context uses it)
            o.group = group.handle.value
        o.rates_now = int(bool(rates_now))  # (rate law: tau of the step's own T, reading 26)
        o.flags = ((BTE_FLAG_PROFILE if profile else 0) | (BTE_FLAG_GENERIC_FACES if generic_faces else 0)
                   | (0 if tma else BTE_FLAG_NO_TMA) | (0 if box else BTE_FLAG_NO_BOX))
        o.max_spare_slabs, o.block_threads, o.band_group = int(max_spare_slabs), int(block_threads), int(band_group)
        o.dir_chunk = int(dir_chunk)
        if cell_part is not None:  # cell partitioning (N3): this rank owns part rank % n_cell_parts
            k["part"] = i32(cell_part)
            assert k["part"].shape == (self.n_cells,)
            o.cell_part, o.n_cell_parts = _p(k["part"]).value, int(n_cell_parts)
        ctx = C.c_void_p()
        _check(lib.bte_create(C.byref(m), C.byref(b), C.byref(d), C.byref(bc), C.byref(o), C.byref(ctx)))
        self.ctx = ctx
        lo, hi = C.c_int32(), C.c_int32()
        _check(lib.bte_band_range(self.ctx, C.byref(lo), C.byref(hi)), self.ctx)
        self.b_lo, self.b_hi = lo.value, hi.value
        self.n_cell_parts = int(n_cell_parts) if cell_part is not None else 1
        self.n_global_cells = self.n_cells
        n = C.c_int64()
        _check(lib.bte_local_cells(self.ctx, C.byref(n), None), self.ctx)
        self.n_cells = n.value  # owned cells (all of them without cell partitioning)

    # -- lifecycle ---------------------------------------------------------------
    def close(self):
        if getattr(self, "ctx", None):
            lib.bte_destroy(self.ctx)
            self.ctx = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    # -- the method --------------------------------------------------------------
    def step(self, dt, n=1):
        _check(lib.bte_step(self.ctx, float(dt), int(n)), self.ctx)

    def step_begin(self, dt):
        _check(lib.bte_step_begin(self.ctx, float(dt)), self.ctx)

    def step_finish(self):
        _check(lib.bte_step_finish(self.ctx), self.ctx)

    def dt_bound(self):
        v = C.c_double()
        _check(lib.bte_dt_bound(self.ctx, C.byref(v)), self.ctx)
        return v.value

    def solve_temperature(self):
        _check(lib.bte_solve_temperature(self.ctx), self.ctx)

    # -- data movement -----------------------------------------------------------
    def temperature(self, out=None):
        out = np.empty(self.n_cells) if out is None else out
        _check(lib.bte_get_temperature(self.ctx, _ptr_any(out)), self.ctx)
        return out

    def temperature_rule(self, rule, out=None):
        """T of the current state under rule 0 (R2), 1 (R1) or 2 (R3), state untouched."""
        out = np.empty(self.n_cells) if out is None else out
        _check(lib.bte_get_temperature_rule(self.ctx, int(rule), _ptr_any(out)), self.ctx)
        return out

    def energy(self):
        out = np.empty(self.n_cells)
        _check(lib.bte_get_energy(self.ctx, _p(out)), self.ctx)
        return out

    def set_energy(self, E):
        E = np.ascontiguousarray(E, np.float64)
        _check(lib.bte_set_energy(self.ctx, _p(E)), self.ctx)

    def intensity(self, b_lo=None, b_hi=None, out=None):
        b_lo = self.b_lo if b_lo is None else b_lo
        b_hi = self.b_hi if b_hi is None else b_hi
        if out is None:
            out = np.empty((b_hi - b_lo, self.n_dirs, self.n_cells))
        _check(lib.bte_get_intensity(self.ctx, int(b_lo), int(b_hi), _ptr_any(out)), self.ctx)
        return out

    def set_intensity(self, I, b_lo=None, b_hi=None):
        b_lo = self.b_lo if b_lo is None else b_lo
        b_hi = self.b_hi if b_hi is None else b_hi
        if isinstance(I, np.ndarray):
            I = np.ascontiguousarray(I, np.float64)
            assert I.shape == (b_hi - b_lo, self.n_dirs, self.n_cells)
        _check(lib.bte_set_intensity(self.ctx, int(b_lo), int(b_hi), _ptr_any(I)), self.ctx)

    def set_equilibrium(self, T):
        T = np.ascontiguousarray(np.broadcast_to(np.asarray(T, np.float64), (self.n_cells,)))
        _check(lib.bte_set_equilibrium(self.ctx, _p(T)), self.ctx)

    # -- cell partitioning (N3) ----------------------------------------------------
    def local_cells(self):
        """Global ids (ascending) of the owned cells; cell-indexed arrays follow this order."""
        ids = np.empty(self.n_cells, np.int64)
        n = C.c_int64()
        _check(lib.bte_local_cells(self.ctx, C.byref(n), _p(ids)), self.ctx)
        return ids

    def halo_size(self, part):
        s, r = C.c_int64(), C.c_int64()
        _check(lib.bte_halo_size(self.ctx, int(part), C.byref(s), C.byref(r)), self.ctx)
        return s.value, r.value

    def halo_export(self, part):
        n, _ = self.halo_size(part)
        buf = np.empty(n)
        if n:
            _check(lib.bte_halo_export(self.ctx, int(part), _p(buf)), self.ctx)
        return buf

    def halo_import(self, part, buf):
        buf = np.ascontiguousarray(buf, np.float64)
        if buf.size:
            _check(lib.bte_halo_import(self.ctx, int(part), _p(buf)), self.ctx)

    def stats(self):
        s = Stats()
        _check(lib.bte_get_stats(self.ctx, C.byref(s)), self.ctx)
        return s.as_dict()

    def reset_stats(self):
        _check(lib.bte_reset_stats(self.ctx), self.ctx)


def _ptr_any(a):
    """Host pointer of a NumPy array or a (pinned, CPU) torch tensor."""
    if isinstance(a, np.ndarray):
        assert a.dtype == np.float64 and a.flags.c_contiguous
        return _p(a)
    if hasattr(a, "data_ptr"):
        assert not a.is_cuda and a.is_contiguous()
        return C.c_void_p(a.data_ptr())
    raise TypeError(type(a))


def solver_from_config(cfg, **kw):
    kw.setdefault("t_init", cfg.t_init)
    kw.setdefault("temp_rule", cfg.temp_rule)
    return Solver(cfg.mesh, cfg.bands, cfg.dirs, cfg.bcs, **kw)


def apply_ic(solver, cfg, seed=None):
    """Seeded IC of the synthetic configs through the public API: equilibrium
    at t_init times the generator's multiplier, then T of that field."""
    from .inputs import SEED, ic_multiplier
    fn = getattr(cfg, "ic_mult", None)
    if not cfg.ic_eps and fn is None:
        return
    seed = SEED if seed is None else seed
    cells = solver.local_cells() if solver.n_cell_parts > 1 else None
    for b in range(solver.b_lo, solver.b_hi):
        I = solver.intensity(b, b + 1)
        mult = (fn(solver.n_dirs, solver.n_global_cells, b) if fn is not None else
                ic_multiplier(solver.n_dirs, solver.n_global_cells, b, cfg.ic_eps, seed))
        I[0] *= mult if cells is None else mult[:, cells]
        solver.set_intensity(I, b, b + 1)
    solver.solve_temperature()
