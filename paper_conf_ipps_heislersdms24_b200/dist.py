"""Band sharding across ranks: process-group plumbing around the C ABI.

One process per GPU (torch.distributed, launched by torch.distributed.run).
The library owns the data-path collective (one NCCL all-reduce of the per-cell
energy per step, L760-763); this module only bootstraps it: rank 0 asks the
library for an NCCL unique id and the process group broadcasts it.
"""
from __future__ import annotations

import os


def band_range(rank: int, world: int, n_bands: int) -> tuple[int, int]:
    """Rows [floor(g nb / P), floor((g+1) nb / P)) of rank g (L773-775); the
    same rule bte_create applies (checked against bte_band_range in the tests)."""
    return rank * n_bands // world, (rank + 1) * n_bands // world


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


def make_solver(cfg, pg=None, **kw):
    """Solver for this rank (world from the process group, if any)."""
    from . import bte
    if pg is None or pg.get_world_size() == 1:
        return bte.solver_from_config(cfg, **kw)
    rank, world = pg.get_rank(), pg.get_world_size()
    return bte.solver_from_config(cfg, rank=rank, world=world, nccl_id=share_nccl_id(pg, rank), **kw)
