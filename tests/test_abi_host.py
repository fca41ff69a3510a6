"""Host-side checks of the C-ABI library (no GPU needed, no compute calls).

libbte.so must load and export every function include/bte.h declares, and
bte_create must reject invalid inputs with BTE_EINVAL during validation,
before it touches a device.
"""
import os
import re
import subprocess

import numpy as np
import pytest

from paper_conf_ipps_heislersdms24_b200 import build as bbuild
from paper_conf_ipps_heislersdms24_b200 import inputs as gen

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def bte():
    bbuild.build()
    from paper_conf_ipps_heislersdms24_b200 import bte as mod
    return mod


def _declared():
    hdr = open(os.path.join(ROOT, "include", "bte.h")).read()
    return sorted(set(re.findall(r"BTE_API\s+[\w\s\*]+?\b(bte_\w+)\s*\(", hdr)))


def test_header_declares_the_north_star_calls():
    names = _declared()
    for must in ("bte_create", "bte_step", "bte_get_temperature", "bte_get_intensity", "bte_destroy"):
        assert must in names


def test_library_exports_every_declared_symbol(bte):
    out = subprocess.check_output(["nm", "-D", "--defined-only", bte.LIB_PATH], text=True)
    exported = {l.split()[-1] for l in out.splitlines() if " T " in l}
    missing = [n for n in _declared() if n not in exported]
    assert not missing, missing
    assert set(bte.EXPORTS) == set(_declared())
    # nothing but the C ABI leaks out
    assert all(n.startswith("bte_") for n in exported if not n.startswith("_")), sorted(exported)[:20]


def test_options_default_and_status_strings(bte):
    o = bte.Options()
    assert bte.lib.bte_options_default(bte.C.byref(o)) == 0
    assert (o.t_init, o.temp_rule, o.newton_rtol, o.newton_max_iter, o.world) == (300.0, 0, 1e-12, 50, 1)
    assert bte.lib.bte_status_string(5) == b"BTE_ENOCONV"


def _small():
    mesh = gen.gen_mesh((4, 3), (1e-6, 1e-6))
    return mesh, gen.gen_bands_si(2), gen.gen_dirs_inplane(8), gen.gen_bcs_fig1(mesh, radius=2e-6)


def _expect_einval(bte, *args, match, **kw):
    with pytest.raises(bte.BTEError) as e:
        bte.Solver(*args, **kw)
    assert e.value.status == bte.BTE_EINVAL, str(e.value)
    assert re.search(match, str(e.value)), str(e.value)


def test_create_validation_rejects_bad_inputs(bte):
    mesh, bands, dirs, bcs = _small()
    bad = dict(mesh, cell_volume=np.where(np.arange(12) == 3, -1.0, mesh["cell_volume"]))
    _expect_einval(bte, bad, bands, dirs, bcs, match="volume")
    bad = dict(mesh, face_area=np.where(np.arange(48) == 7, 0.0, mesh["face_area"]))
    _expect_einval(bte, bad, bands, dirs, bcs, match="area")
    nrm = mesh["face_normal"].copy()
    nrm[5] *= 1.1
    _expect_einval(bte, dict(mesh, face_normal=nrm), bands, dirs, bcs, match="normal")
    nrm = mesh["face_normal"].copy()
    nrm[5] = [0.6, 0.0, 0.8]
    _expect_einval(bte, dict(mesh, face_normal=nrm), bands, dirs, bcs, match="n_z")
    _expect_einval(bte, dict(mesh, dim=4), bands, dirs, bcs, match="dim")
    b2 = dict(bands, tau=np.array([1e-11, -1.0]))
    _expect_einval(bte, mesh, b2, dirs, bcs, match="tau")
    b3 = dict(bands, tau=np.array([np.inf, np.inf]))
    _expect_einval(bte, mesh, b3, dirs, bcs, match="weights are zero")
    d2 = dict(dirs, w=-dirs["w"])
    _expect_einval(bte, mesh, bands, d2, bcs, match="weight")
    _expect_einval(bte, mesh, bands, gen.gen_dirs_inplane(7), bcs, match="reflection")
    b4 = dict(bcs, kind=np.full(bcs["n_bfaces"], 7, np.int32))
    _expect_einval(bte, mesh, bands, dirs, b4, match="kind")
    nbr = mesh["face_nbr"].copy()
    nbr[0] = 99
    _expect_einval(bte, dict(mesh, face_nbr=nbr), bands, dirs, bcs, match="out of range")
    _expect_einval(bte, mesh, bands, dirs, bcs, match="rank", rank=2, world=2)
    _expect_einval(bte, mesh, bands, dirs, bcs, match="owns no band", rank=0, world=3)


def test_last_error_without_context(bte):
    mesh, bands, dirs, bcs = _small()
    with pytest.raises(bte.BTEError):
        bte.Solver(dict(mesh, dim=1), bands, dirs, bcs)
    assert b"dim" in bte.lib.bte_last_error(None)
