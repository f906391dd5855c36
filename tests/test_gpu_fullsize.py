"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py
times (same library defaults: tile, TMA ring, segments, CUDA graphs).

One step of a node depends only on the moments of its 3x3(x3) neighbourhood,
so the oracle can compute sampled outputs one by one: for each sampled node
it runs one step on the neighbourhood box (domain faces where the box touches
them; periodic wrap along uncut periodic axes; a wall at the far end of a box
clipped by a domain face, so nothing reaches the centre through a face the
domain does not have) and the centre's moments must match the GPU's.
Samples: seeded random nodes plus every corner, edge midpoint and face centre.
Multi-step behaviour at full size is checked through invariants (mass and
momentum) that hold at any size."""
import itertools

import numpy as np
import pytest

from parity import TOL
from paper_conf_sc_valero_laravgr23_b200 import configs

pytestmark = pytest.mark.gpu

FACES = ("x-", "x+", "y-", "y+", "z-", "z+")


def cfg(name):
    if name == "C2-fp64":
        return configs.c2("fp64")
    if name == "C2-fp32":
        return configs.c2("fp32")
    if name == "C3":
        return configs.c3()
    if name == "C4":
        return configs.c4()
    if name == "C5w":  # weak-scaling per-GPU shape of C5: 1024 x 1024 x 128
        return configs.c5(nz=128)
    raise KeyError(name)


def sample_nodes(shape, rng, n=48):
    """shape = grid (nz, ny, nx) or (ny, nx); returns index tuples in grid order."""
    pts = {tuple(int(rng.integers(0, s)) for s in shape) for _ in range(n)}
    for corner in itertools.product(*[(0, s - 1) for s in shape]):
        pts.add(corner)
    for ax in range(len(shape)):  # face centres and edge midpoints
        for side in (0, shape[ax] - 1):
            p = [s // 2 for s in shape]
            p[ax] = side
            pts.add(tuple(p))
            for ax2 in range(len(shape)):
                if ax2 != ax:
                    q = list(p)
                    q[ax2] = 0
                    pts.add(tuple(q))
    return sorted(pts)


def neighbourhood(c, m0, p):
    """(moments of the box, box dims (nx,ny,nz), box boundary, centre index in box grid)."""
    D = c.D
    grid = m0.shape[1:]                    # (nz, ny, nx) or (ny, nx)
    idx, centre, faces = [], [], {}
    for g, n in enumerate(grid):
        a = D - 1 - g                       # physical axis of grid axis g
        lo_kind = c.boundary.get(FACES[2 * a], {"kind": "periodic"})
        hi_kind = c.boundary.get(FACES[2 * a + 1], {"kind": "periodic"})
        pg = p[g]
        if lo_kind["kind"] == "periodic":
            ids = [(pg - 1) % n, pg, (pg + 1) % n]
            centre.append(1)
        else:
            lo, hi = max(pg - 1, 0), min(pg + 1, n - 1)
            ids = list(range(lo, hi + 1))
            centre.append(pg - lo)
            # the box face on a domain face takes its kind; the other end of a
            # clipped (2-wide) box is a wall, so that nothing wraps onto the
            # centre through a box face the real domain does not have
            faces[FACES[2 * a]] = dict(lo_kind) if pg == 0 else {"kind": "wall"}
            faces[FACES[2 * a + 1]] = dict(hi_kind) if pg == n - 1 else {"kind": "wall"}
        idx.append(ids)
    box = m0[np.ix_(range(m0.shape[0]), *idx)]
    # open-face profiles: cut the face-node array to the box
    for name, spec in faces.items():
        prof = spec.get("u_profile")
        if prof is not None:
            a = FACES.index(name) // 2
            others = [g for g in range(D) if D - 1 - g != a]  # grid axes of the face array, slower first
            sub = np.asarray(prof)
            sub = sub[np.ix_(*[idx[g] for g in others], range(sub.shape[-1]))]
            spec["u_profile"] = sub.reshape(-1, sub.shape[-1])
    dims = tuple(len(ids) for ids in idx)[::-1]  # physical (nx, ny[, nz])
    return box, dims, faces, tuple(centre)


@pytest.mark.parametrize("name", ["C2-fp64", "C2-fp32", "C3", "C4", "C5w"])
def test_fullsize_one_step_sampled(name):
    import oracle
    from paper_conf_sc_valero_laravgr23_b200 import mrlbm
    c = cfg(name)
    m0 = c.initial_moments()
    with mrlbm.Solver(c.lattice, c.nx, c.ny, c.nz, c.tau, c.regularization, c.boundary,
                      precision=c.precision) as s:
        s.set_moments(m0)
        s.step(1)
        got = s.get_moments()
    rng = np.random.default_rng(7)
    pts = sample_nodes(m0.shape[1:], rng)
    ref_vals, gpu_vals = [], []
    for p in pts:
        box, dims, faces, ctr = neighbourhood(c, m0, p)
        nz = dims[2] if c.D == 3 else 1
        o = oracle.Oracle(c.lattice, dims[0], dims[1], nz, c.tau, c.regularization, faces)
        o.set_moments(box)
        o.step(1)
        ref_vals.append(o.get_moments()[(slice(None),) + ctr])
        gpu_vals.append(got[(slice(None),) + tuple(p)])
    ref, gv = np.array(ref_vals).T, np.array(gpu_vals).T
    D = c.D
    groups = {"rho": [0], "u": list(range(1, 1 + D)), "Pi": list(range(1 + D, ref.shape[0]))}
    tol = {"fp64": 1e-13, "fp32": 1e-5}[c.precision]
    for g, ix in groups.items():
        den = max(np.abs(ref[ix]).max(), 1e-300)
        err = np.abs(gv[ix] - ref[ix]).max() / den
        assert err <= tol, f"{name} {g}: {err} over {len(pts)} sampled nodes"


@pytest.mark.parametrize("name", ["C2-fp64", "C2-fp32", "C3", "C4"])
def test_fullsize_invariants(name):
    """Mass (closed cavities, periodic box) and momentum (periodic box) over
    200 steps at full size, through the bench's CUDA-graph step path."""
    from paper_conf_sc_valero_laravgr23_b200 import mrlbm
    c = cfg(name)
    m0 = c.initial_moments()
    D = c.D
    with mrlbm.Solver(c.lattice, c.nx, c.ny, c.nz, c.tau, c.regularization, c.boundary,
                      precision=c.precision) as s:
        s.set_moments(m0)
        s.step(200)
        s.check_finite()
        m1 = s.get_moments()
    mass0, mass1 = m0[0].sum(dtype=np.float64), m1[0].sum(dtype=np.float64)
    tol = TOL[c.precision] * 10
    assert abs(mass1 - mass0) / mass0 < tol
    if not c.boundary:  # fully periodic (C3): momentum too
        for a in range(D):
            p0 = (m0[0] * m0[1 + a]).sum()
            p1 = (m1[0] * m1[1 + a]).sum()
            assert abs(p1 - p0) / mass0 < tol
