"""Small runs of every flux-kernel variant, for compute-sanitizer (memcheck,
racecheck, synccheck).  Exits non-zero on any library error."""
import dataclasses
import sys

sys.path.insert(0, ".")
from paper_conf_ipps_heislersdms24_b200 import bte, inputs as gen  # noqa: E402


def run(cfg, **kw):
    with bte.solver_from_config(cfg, **kw) as s:
        bte.apply_ic(s, cfg)
        s.step(cfg.dt, 2)
        s.temperature()
        return bte.FLUX_VARIANTS[s.stats()["flux_variant"]]


c3d = gen.small_3d_config((13, 7, 5), n_spectral=3, ntheta=4, nphi=8)
c1 = dataclasses.replace(gen.make_config("C1"), nsteps=2)
mesh = gen.gen_mesh((40, 24), (1e-6, 1e-6))
bands, dirs = gen.gen_bands_si(3), gen.gen_dirs_product(4, 8)
cst = gen.Config("st", mesh, bands, dirs, gen.gen_bcs_fig1(mesh, radius=3e-6), 300.0,
                 0.5 * gen.cartesian_dt_bound(mesh, bands, dirs), 2, ic_eps=0.2)
for name, cfg, kw in [("C1", c1, {}), ("3d-tma", c3d, {}), ("3d-tma-bg1", c3d, {"band_group": 1}),
                      ("3d-reg", c3d, {"tma": False}), ("3d-generic", c3d, {"generic_faces": True}),
                      ("stencil", cst, {"stencil": True}), ("rotation", c3d, {"max_spare_slabs": 2})]:
    print(name, run(cfg, **kw), flush=True)
print("ALL OK")
