"""Band sharding across ranks: process-group plumbing around the C ABI.

One process per GPU (torch.distributed, launched by torch.distributed.run).
The library owns the data-path collectives (reduce-scatter of the per-cell
energy and all-gather of T per step, L760-763); this module only bootstraps
them: rank 0 asks the library for an NCCL unique id and the process group
broadcasts it.  (Ranks that are threads of one process use bte.Group instead.)
"""
from __future__ import annotations

import os


def band_range(rank: int, world: int, n_bands: int) -> tuple[int, int]:
    """Rows [floor(g nb / P), floor((g+1) nb / P)) of rank g (L773-775); the
    same rule bte_create applies (checked against bte_band_range in the tests)."""
    return rank * n_bands // world, (rank + 1) * n_bands // world


def rank_grid(rank: int, world: int, n_cell_parts: int = 1) -> tuple[int, int]:
    """(cell part, band group) of a rank under cell partitioning (SURVEY 8(f)
    N3): part = rank % P, group = rank // P; the rule bte_create applies."""
    assert world % n_cell_parts == 0
    return rank % n_cell_parts, rank // n_cell_parts


def partition_cells(centres, n_parts: int):
    """Recursive coordinate bisection of the cells (a Metis-style partition
    without the library dependency; the paper partitions its meshes with Metis,
    L728-735): split the cell set at the median of its longest extent, in
    proportion to the parts on each side, until every part has its cells.
    Deterministic (ties broken by cell id); parts are spatially compact, so a
    part's halo is its surface.  Returns part[n_cells] (int32)."""
    import numpy as np
    x = np.asarray(centres, dtype=np.float64)
    out = np.zeros(x.shape[0], np.int32)

    def rec(ids, p0, n):
        if n == 1:
            out[ids] = p0
            return
        ext = x[ids].max(axis=0) - x[ids].min(axis=0)
        ax = int(np.argmax(ext))
        order = ids[np.lexsort((ids, x[ids, ax]))]
        nl = n // 2
        k = int(round(len(ids) * nl / n))
        rec(order[:k], p0, nl)
        rec(order[k:], p0 + nl, n - nl)

    rec(np.arange(x.shape[0]), 0, int(n_parts))
    return out


def slab_partition(centres, n_parts: int, axis: int = 2):
    """Slabs of whole cell layers along one axis (equal cell counts up to a
    layer): on the paper's structured 3-D grids, z slabs keep the box kernel
    (bte_options.cell_part, DESIGN.md 9 N3).  Returns part[n_cells] (int32)."""
    import numpy as np
    x = np.asarray(centres, dtype=np.float64)[:, axis]
    levels = np.unique(x)
    layer = np.searchsorted(levels, x)
    counts = np.bincount(layer, minlength=levels.size)
    cum = np.cumsum(counts) - counts  # cells before each layer
    part_of_layer = np.minimum(n_parts - 1, (cum * n_parts) // x.size).astype(np.int32)
    return part_of_layer[layer]


def env_rank_world():
    return (int(os.environ.get("RANK", "0")), int(os.environ.get("WORLD_SIZE", "1")),
            int(os.environ.get("LOCAL_RANK", "0")))


def share_nccl_id(pg, rank: int, make_id=None) -> bytes:
    """Rank 0 creates the 128-byte NCCL id, every rank returns it."""
    if make_id is None:
        from . import bte
        make_id = bte.nccl_unique_id
    obj = [make_id() if rank == 0 else None]
    pg.broadcast_object_list(obj, src=0)
    nid = obj[0]
    assert isinstance(nid, (bytes, bytearray)) and len(nid) == 128
    return bytes(nid)


def make_solver(cfg, pg=None, n_cell_parts=1, **kw):
    """Solver for this rank (world from the process group, if any).
    n_cell_parts > 1: cell partitioning (N3) -- z slabs on 3-D meshes (the box
    kernel keeps running on structured grids), coordinate bisection on 2-D --
    combined with band sharding over world / n_cell_parts groups."""
    from . import bte
    if n_cell_parts > 1:
        cen = cfg.mesh["cell_centre"]
        parts = slab_partition(cen, n_cell_parts) if cfg.mesh["dim"] == 3 else partition_cells(cen, n_cell_parts)
        kw.update(cell_part=parts, n_cell_parts=n_cell_parts)
    kw.setdefault("device", env_rank_world()[2])  # (one process per GPU: this rank's LOCAL_RANK)
    if pg is None or pg.get_world_size() == 1:
        return bte.solver_from_config(cfg, **kw)
    rank, world = pg.get_rank(), pg.get_world_size()
    return bte.solver_from_config(cfg, rank=rank, world=world, nccl_id=share_nccl_id(pg, rank), **kw)
