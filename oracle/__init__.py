"""ctypes wrapper of the CPU oracle (TEST INFRASTRUCTURE ONLY).

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
``--impl reference`` legs may import this package.  The product path
(paper_conf_ipps_heislersdms24_b200) never imports it, and it never takes an
input from the CUDA path.  See bte_oracle.h for the method and citations.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "bte_oracle.c")
_HDR = os.path.join(_HERE, "bte_oracle.h")
_LIB = os.path.join(_HERE, "liboracle.so")

OK, EINVAL, ENOCONV = 0, 1, 5


def build(force=False):
    """Compile liboracle.so with gcc (plain -O2, no fast-math, OpenMP)."""
    stale = (not os.path.exists(_LIB) or
             os.path.getmtime(_LIB) < max(os.path.getmtime(_SRC), os.path.getmtime(_HDR)))
    if force or stale:
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-fno-fast-math", "-shared", "-fPIC",
                               _SRC, "-o", _LIB, "-lm"])
    return _LIB


class _Problem(C.Structure):
    _fields_ = [
        ("dim", C.c_int32), ("n_cells", C.c_int64),
        ("face_offsets", C.c_void_p), ("face_nbr", C.c_void_p), ("face_area", C.c_void_p),
        ("face_normal", C.c_void_p), ("cell_volume", C.c_void_p),
        ("n_bands", C.c_int32), ("omega", C.c_void_p), ("vg", C.c_void_p), ("tau", C.c_void_p),
        ("C", C.c_void_p),
        ("n_dirs", C.c_int32), ("s", C.c_void_p), ("w", C.c_void_p),
        ("n_bfaces", C.c_int64), ("bkind", C.c_void_p), ("t_wall", C.c_void_p),
        ("temp_rule", C.c_int32), ("newton_rtol", C.c_double), ("newton_maxit", C.c_int32),
        ("rate_a", C.c_void_p), ("rate_b", C.c_void_p), ("rate_theta", C.c_void_p),
        ("rates_now", C.c_int32),
    ]


_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = C.CDLL(build())
        P = C.POINTER(_Problem)
        vp, i32, i64, dbl = C.c_void_p, C.c_int32, C.c_int64, C.c_double
        _lib.oracle_I0.argtypes = [dbl, dbl, dbl]
        _lib.oracle_I0.restype = dbl
        _lib.oracle_weight.argtypes = [P, i32]
        _lib.oracle_weight.restype = dbl
        _lib.oracle_weight_at.argtypes = [P, i32, dbl]
        _lib.oracle_weight_at.restype = dbl
        _lib.oracle_rate.argtypes = [P, i32, dbl]
        _lib.oracle_rate.restype = dbl
        _lib.oracle_reflection_map.argtypes = [P, vp]
        _lib.oracle_update_intensity.argtypes = [P, vp, vp, vp, vp, vp, dbl, i32, i32]
        _lib.oracle_update_intensity.restype = None
        _lib.oracle_energy.argtypes = [P, vp, vp, i32, i32, vp]
        _lib.oracle_energy.restype = None
        _lib.oracle_newton.argtypes = [P, vp, vp, vp, vp]
        _lib.oracle_equilibrium.argtypes = [P, vp, i32, i32, vp]
        _lib.oracle_equilibrium.restype = None
        _lib.oracle_run.argtypes = [P, dbl, i64, vp, vp, vp]
        _lib.oracle_step_cells_equilibrium.argtypes = [P, vp, vp, vp, i64, dbl, vp, vp]
        _lib.oracle_energy_subset.argtypes = [P, i64, vp, vp, vp]
        _lib.oracle_energy_subset.restype = None
        _lib.oracle_newton_subset.argtypes = [P, i64, vp, vp, vp]
        _lib.oracle_step_subset.argtypes = [P, vp, i64, vp, vp, vp, vp, i64, vp, dbl, vp, vp]
    return _lib


def _ptr(a):
    return a.ctypes.data_as(C.c_void_p)


def _optr(a):
    """Pointer of an optional per-cell array (None -> NULL)."""
    return None if a is None else _ptr(a)


def _cells(x, nc):
    return None if x is None else np.ascontiguousarray(np.broadcast_to(np.asarray(x, np.float64), (nc,)))


class Problem:
    """A mesh + band table + direction set + BCs as the oracle sees them."""

    def __init__(self, mesh, bands, dirs, bcs, temp_rule=0, rtol=1e-12, maxit=50, rates_now=False):
        f64 = lambda x: np.ascontiguousarray(x, dtype=np.float64)
        i64 = lambda x: np.ascontiguousarray(x, dtype=np.int64)
        i32 = lambda x: np.ascontiguousarray(x, dtype=np.int32)
        self.keep = dict(
            face_offsets=i64(mesh["face_offsets"]), face_nbr=i64(mesh["face_nbr"]),
            face_area=f64(mesh["face_area"]), face_normal=f64(mesh["face_normal"]),
            cell_volume=f64(mesh["cell_volume"]),
            omega=f64(bands["omega"]), vg=f64(bands["vg"]), tau=f64(bands["tau"]), C=f64(bands["C"]),
            s=f64(dirs["s"]), w=f64(dirs["w"]),
            bkind=i32(bcs["kind"]), t_wall=f64(bcs["t_wall"]),
        )
        # temperature-dependent relaxation times (N1): 1/tau_b(T) = a + b T exp(-theta/T)
        self.has_rates = bands.get("rate_a") is not None
        if self.has_rates:
            self.keep.update(rate_a=f64(bands["rate_a"]), rate_b=f64(bands["rate_b"]),
                             rate_theta=f64(bands["rate_theta"]))
        k = self.keep
        self.nc, self.nb, self.nd = int(mesh["n_cells"]), int(bands["n_bands"]), int(dirs["n_dirs"])
        self.nbf = int(bcs["n_bfaces"])
        self.s = _Problem(
            dim=int(mesh["dim"]), n_cells=self.nc,
            face_offsets=_ptr(k["face_offsets"]).value, face_nbr=_ptr(k["face_nbr"]).value,
            face_area=_ptr(k["face_area"]).value, face_normal=_ptr(k["face_normal"]).value,
            cell_volume=_ptr(k["cell_volume"]).value,
            n_bands=self.nb, omega=_ptr(k["omega"]).value, vg=_ptr(k["vg"]).value,
            tau=_ptr(k["tau"]).value, C=_ptr(k["C"]).value,
            n_dirs=self.nd, s=_ptr(k["s"]).value, w=_ptr(k["w"]).value,
            n_bfaces=self.nbf, bkind=_ptr(k["bkind"]).value, t_wall=_ptr(k["t_wall"]).value,
            temp_rule=int(temp_rule), newton_rtol=float(rtol), newton_maxit=int(maxit),
            rate_a=_ptr(k["rate_a"]).value if self.has_rates else None,
            rate_b=_ptr(k["rate_b"]).value if self.has_rates else None,
            rate_theta=_ptr(k["rate_theta"]).value if self.has_rates else None,
            rates_now=int(bool(rates_now)),
        )
        self._r = None

    @property
    def ref(self):
        return C.byref(self.s)

    # -- pieces of the method -------------------------------------------------
    def I0(self, b, T):
        return lib().oracle_I0(float(self.keep["C"][b]), float(self.keep["omega"][b]), float(T))

    def weight(self, b):
        return lib().oracle_weight(self.ref, int(b))

    def weights(self):
        return np.array([self.weight(b) for b in range(self.nb)])

    def weight_at(self, b, Tr):
        return lib().oracle_weight_at(self.ref, int(b), float(Tr))

    def rate(self, b, Tr):
        """1/tau_b at rate temperature Tr (constant rates ignore Tr)."""
        return lib().oracle_rate(self.ref, int(b), float(Tr))

    def _need_tr(self, Tr):
        if self.has_rates and Tr is None:
            raise ValueError("temperature-dependent rates need the rate temperature Tr")
        return _cells(Tr, self.nc)

    def reflection_map(self):
        if self._r is None:
            r = np.empty((max(self.nbf, 1), self.nd), dtype=np.int32)
            rc = lib().oracle_reflection_map(self.ref, _ptr(r))
            if rc != OK:
                raise ValueError("specular reflection not closed on the direction set")
            self._r = r
        return self._r

    def equilibrium(self, T, b_lo=0, b_hi=None):
        b_hi = self.nb if b_hi is None else b_hi
        T = np.ascontiguousarray(np.broadcast_to(np.asarray(T, np.float64), (self.nc,)))
        I = np.empty((b_hi - b_lo, self.nd, self.nc))
        lib().oracle_equilibrium(self.ref, _ptr(T), int(b_lo), int(b_hi), _ptr(I))
        return I

    def update_intensity(self, T, I, dt, b_lo=0, b_hi=None, Tr=None):
        b_hi = self.nb if b_hi is None else b_hi
        T = np.ascontiguousarray(T, np.float64)
        I = np.ascontiguousarray(I, np.float64)
        Tr = self._need_tr(Tr)
        out = np.zeros_like(I)
        lib().oracle_update_intensity(self.ref, _ptr(self.reflection_map()), _ptr(T), _optr(Tr), _ptr(I),
                                      _ptr(out), float(dt), int(b_lo), int(b_hi))
        return out

    def energy(self, I, b_lo=0, b_hi=None, Tr=None):
        b_hi = self.nb if b_hi is None else b_hi
        I = np.ascontiguousarray(I, np.float64)
        Tr = self._need_tr(Tr)
        E = np.empty(self.nc)
        lib().oracle_energy(self.ref, _ptr(I), _optr(Tr), int(b_lo), int(b_hi), _ptr(E))
        return E

    def newton(self, E, T_guess, Tr=None):
        E = np.ascontiguousarray(E, np.float64)
        Tr = self._need_tr(Tr)
        T = np.array(np.broadcast_to(np.asarray(T_guess, np.float64), (self.nc,)))
        iters = np.zeros(self.nc, dtype=np.int32)
        rc = lib().oracle_newton(self.ref, _ptr(E), _optr(Tr), _ptr(T), _ptr(iters))
        if rc != OK:
            raise RuntimeError(f"oracle newton failed rc={rc}")
        return T, iters

    def run(self, I, T, dt, nsteps, Tr=None):
        """nsteps explicit steps from (I, T); returns new copies.  With a rate
        law the state also carries the rate temperature Tr: pass it and get
        (I, T, Tr) back."""
        I = np.array(I, dtype=np.float64, order="C")
        T = np.array(T, dtype=np.float64, order="C")
        Tr_in = Tr
        Tr = None if Tr is None else np.array(np.broadcast_to(np.asarray(Tr, np.float64), (self.nc,)))
        self._need_tr(Tr)
        assert I.shape == (self.nb, self.nd, self.nc)
        self.reflection_map()  # raise early on an unclosed map
        rc = lib().oracle_run(self.ref, float(dt), int(nsteps), _ptr(I), _ptr(T), _optr(Tr))
        if rc != OK:
            raise RuntimeError(f"oracle run failed rc={rc}")
        return (I, T) if Tr_in is None else (I, T, Tr)

    def step_cells_equilibrium(self, T0, cells, dt):
        T0 = np.ascontiguousarray(T0, np.float64)
        cells = np.ascontiguousarray(cells, np.int64)
        out = np.empty((cells.size, self.nb, self.nd))
        T1 = np.empty(cells.size)
        rc = lib().oracle_step_cells_equilibrium(self.ref, _ptr(self.reflection_map()), _ptr(T0),
                                                 _ptr(cells), int(cells.size), float(dt),
                                                 _ptr(out), _ptr(T1))
        if rc != OK:
            raise RuntimeError(f"oracle sampled step failed rc={rc}")
        return out, T1

    def run_until_failure(self, I, T, dt, nsteps, Tr=None):
        """Up to nsteps steps, one at a time; stops after the step whose
        temperature solve fails (ENOCONV, the state of that step: the failed
        cells keep their previous T).  Returns (I, T, Tr, steps_taken, rc)."""
        I = np.array(I, dtype=np.float64, order="C")
        T = np.array(T, dtype=np.float64, order="C")
        Tr = None if Tr is None else np.array(np.broadcast_to(np.asarray(Tr, np.float64), (self.nc,)))
        self._need_tr(Tr)
        self.reflection_map()
        rc, k = OK, 0
        while k < nsteps and rc == OK:
            rc = lib().oracle_run(self.ref, float(dt), 1, _ptr(I), _ptr(T), _optr(Tr))
            k += 1
        return I, T, Tr, k, rc

    # -- subsets of cells (sampled checks of full fields) ------------------------
    def subset_initial(self, sub, I_sub, T_guess, Tr_sub=None):
        """T of the subset cells' intensities I_sub[b][d][k] (Newton from T_guess)."""
        sub = np.ascontiguousarray(sub, np.int64)
        I_sub = np.ascontiguousarray(I_sub, np.float64)
        Tr = None if Tr_sub is None else np.ascontiguousarray(np.broadcast_to(np.asarray(Tr_sub, np.float64), sub.shape))
        E = np.empty(sub.size)
        lib().oracle_energy_subset(self.ref, int(sub.size), _ptr(I_sub), _optr(Tr), _ptr(E))
        T = np.array(np.broadcast_to(np.asarray(T_guess, np.float64), sub.shape))
        rc = lib().oracle_newton_subset(self.ref, int(sub.size), _ptr(E), _optr(Tr), _ptr(T))
        if rc != OK:
            raise RuntimeError(f"oracle subset newton failed rc={rc}")
        return T

    def step_subset(self, sub, I_sub, T_sub, sel, dt, Tr_sub=None):
        """One step of cells sub[sel] from a subset state (neighbours in sub)."""
        sub = np.ascontiguousarray(sub, np.int64)
        sel = np.ascontiguousarray(sel, np.int64)
        I_sub = np.ascontiguousarray(I_sub, np.float64)
        T_sub = np.ascontiguousarray(T_sub, np.float64)
        Tr = None if Tr_sub is None else np.ascontiguousarray(Tr_sub, np.float64)
        out = np.empty((sel.size, self.nb, self.nd))
        T1 = np.empty(sel.size)
        rc = lib().oracle_step_subset(self.ref, _ptr(self.reflection_map()), int(sub.size), _ptr(sub), _ptr(I_sub),
                                      _ptr(T_sub), _optr(Tr), int(sel.size), _ptr(sel), float(dt), _ptr(out),
                                      _ptr(T1))
        if rc != OK:
            raise RuntimeError(f"oracle subset step failed rc={rc}")
        return out, T1

    # -- initial state ----------------------------------------------------------
    def initial_state(self, t_init, ic_eps=0.0, seed=None, mult_fn=None, with_tr=False):
        """IC of the synthetic configs: I = I0_b(t_init) * multiplier, then
        T = temperature of that field (Newton from t_init, weights at the rate
        temperature Tr = t_init).  with_tr: also return Tr."""
        T = np.full(self.nc, float(t_init))
        Tr = np.full(self.nc, float(t_init)) if (with_tr or self.has_rates) else None
        I = self.equilibrium(T)
        if ic_eps or mult_fn is not None:
            from paper_conf_ipps_heislersdms24_b200.inputs import ic_multiplier, SEED
            for b in range(self.nb):
                I[b] *= (mult_fn(self.nd, self.nc, b) if mult_fn is not None else
                         ic_multiplier(self.nd, self.nc, b, ic_eps, SEED if seed is None else seed))
            T, _ = self.newton(self.energy(I, Tr=Tr), T, Tr=Tr)
        return (I, T, Tr) if with_tr else (I, T)


def problem_from_config(cfg, **kw):
    return Problem(cfg.mesh, cfg.bands, cfg.dirs, cfg.bcs, temp_rule=cfg.temp_rule, **kw)
