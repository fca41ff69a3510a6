"""Small runs of every flux-kernel variant (and the halo pack / unpack of a
cell-partitioned run), for compute-sanitizer (memcheck, racecheck, synccheck):
bash tools/gpu_sanitize.sh.  Exits non-zero on any library error."""
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
box3 = gen.small_3d_config((34, 9, 5), n_spectral=3)
law = gen.with_rate_law(box3.bands)
box3law = dataclasses.replace(box3, bands=law, dt=0.5 * gen.cartesian_dt_bound(box3.mesh, law, box3.dirs, t_max=350.0))
law2 = gen.with_rate_law(cst.bands)
cstlaw = dataclasses.replace(cst, bands=law2, dt=0.5 * gen.cartesian_dt_bound(cst.mesh, law2, cst.dirs, t_max=350.0))
c6t = dataclasses.replace(gen.make_config("C6t"), nsteps=2)


def run_parts(cfg, n_parts, slabs=False):
    from paper_conf_ipps_heislersdms24_b200.dist import partition_cells, slab_partition
    parts = (slab_partition if slabs else partition_cells)(cfg.mesh["cell_centre"], n_parts)
    ss = [bte.solver_from_config(cfg, rank=r, world=n_parts, cell_part=parts, n_cell_parts=n_parts)
          for r in range(n_parts)]
    try:
        for _ in range(2):
            bufs = {(a, b): ss[a].halo_export(b) for a in range(n_parts) for b in range(n_parts) if a != b}
            for (a, b), buf in bufs.items():
                ss[b].halo_import(a, buf)
            for s in ss:
                s.step_begin(cfg.dt)
            for s in ss:
                s.step_finish()
        return bte.FLUX_VARIANTS[ss[0].stats()["flux_variant"]]
    finally:
        for s in ss:
            s.close()


def run_group(cfg, world, n_parts=1):
    """world ranks as threads on one in-process group (bte_group_create):
    the band-sharded / cell-partitioned step through bte_step."""
    import threading
    from paper_conf_ipps_heislersdms24_b200.dist import partition_cells
    kw = {}
    if n_parts > 1:
        kw = dict(cell_part=partition_cells(cfg.mesh["cell_centre"], n_parts), n_cell_parts=n_parts)
    err = []
    with bte.Group(world) as g:
        def rank(r):
            try:
                with bte.solver_from_config(cfg, rank=r, world=world, group=g, **kw) as s:
                    bte.apply_ic(s, cfg)
                    s.step(cfg.dt, 2)
                    s.temperature()
            except Exception as e:  # noqa: BLE001
                err.append(e)
        ts = [threading.Thread(target=rank, args=(r,)) for r in range(world)]
        [t.start() for t in ts]
        [t.join() for t in ts]
    if err:
        raise err[0]
    return "ok"


def run_enoconv(**kw):
    cfg = gen.failing_strip_config()
    with bte.solver_from_config(cfg, **kw) as s:
        bte.apply_ic(s, cfg)
        try:
            s.step(cfg.dt, cfg.nsteps)
        except bte.BTEError as e:
            assert e.status == bte.BTE_ENOCONV and s.stats()["steps"] == 4
            return "enoconv at step 4"
    raise AssertionError("no ENOCONV")


print("group-band-3", run_group(c3d, 3), flush=True)
print("group-hybrid-2x2", run_group(dataclasses.replace(gen.make_config("C2"), nsteps=2), 4, n_parts=2), flush=True)
print("enoconv-graph", run_enoconv(), flush=True)
print("enoconv-profile", run_enoconv(profile=True), flush=True)
print("parts-3d", run_parts(c3d, 3), flush=True)
print("parts-zslab-box", run_parts(box3, 2, slabs=True), flush=True)
print("parts-tri", run_parts(c6t, 2), flush=True)
for name, cfg, kw in [("C1", c1, {}), ("box3d", box3, {}), ("box3d-law", box3law, {}), ("box2d", cst, {}),
                      ("box2d-law", cstlaw, {}), ("box2d-rotation", cst, {"max_spare_slabs": 2}),
                      ("triangles", c6t, {}), ("3d-tma", c3d, {}), ("3d-tma-bg1", c3d, {"band_group": 1}),
                      ("3d-reg", c3d, {"tma": False}), ("3d-generic", c3d, {"generic_faces": True}),
                      ("2d-tma", cst, {"box": False}), ("rotation", c3d, {"max_spare_slabs": 2})]:
    print(name, run(cfg, **kw), flush=True)
print("ALL OK")
