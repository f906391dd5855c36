"""Host-side helpers for the slab decomposition (no arithmetic of the method).

The library owns rank r's contiguous slab of the sweep axis (z in 3D, y in
2D); these helpers cut a global ABI moment array into slabs and gather the
slabs back with torch.distributed (any backend; gloo in the CPU tests)."""
from __future__ import annotations

import numpy as np


def slab_bounds(n_global: int, nranks: int, rank: int):
    """(offset, n_local) -- must agree with mrlbm_partition (remainder to the first ranks)."""
    q, r = divmod(n_global, nranks)
    n_local = q + (1 if rank < r else 0)
    offset = rank * q + min(rank, r)
    return offset, n_local


def slab_of(global_moments: np.ndarray, nranks: int, rank: int) -> np.ndarray:
    """Rank's slab of a global [M][nz][ny][nx] (2D: [M][ny][nx]) array: axis 1 is the slab axis."""
    off, n = slab_bounds(global_moments.shape[1], nranks, rank)
    return np.ascontiguousarray(global_moments[:, off:off + n])


def gather_slabs(local: np.ndarray, n_global: int, group=None) -> np.ndarray:
    """All-gather every rank's slab into the global array (torch.distributed)."""
    import torch
    import torch.distributed as dist
    world = dist.get_world_size(group)
    shapes = [slab_bounds(n_global, world, r)[1] for r in range(world)]
    nmax = max(shapes)
    buf = np.zeros((local.shape[0], nmax) + local.shape[2:], dtype=local.dtype)
    buf[:, :local.shape[1]] = local
    t = torch.from_numpy(buf)
    out = [torch.empty_like(t) for _ in range(world)]
    dist.all_gather(out, t, group=group)
    return np.concatenate([o.numpy()[:, :shapes[r]] for r, o in enumerate(out)], axis=1)


def slab_neighbours(nranks: int, rank: int, periodic: bool):
    """(lower, upper) neighbour ranks along the slab axis, None at a bounded end
    (the library's own rule: periodic slab axis wraps rank 0 <-> rank P-1)."""
    lo = rank - 1 if rank > 0 else (nranks - 1 if periodic else None)
    hi = rank + 1 if rank < nranks - 1 else (0 if periodic else None)
    return lo, hi


def slab_axis_periodic(boundary: dict | None, D: int) -> bool:
    """Missing faces are periodic (include/mrlbm.h); the slab axis is z (3D) / y (2D)."""
    face = "z-" if D == 3 else "y-"
    spec = (boundary or {}).get(face)
    return spec is None or spec.get("kind", "periodic") == "periodic"


def p2p_connect(solver, handles: list, periodic: bool):
    """Connect a P2P-transport solver to its slab neighbours, given every rank's
    mrlbm_p2p_handle blob (e.g. from torch.distributed.all_gather_object)."""
    lo, hi = slab_neighbours(len(handles), solver.rank, periodic)
    solver.p2p_connect(handles[lo] if lo is not None else None, handles[hi] if hi is not None else None)
