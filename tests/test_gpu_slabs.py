"""Slab decomposition on one GPU (slab-group mode: the kernels, ghost planes
and interior/boundary launch split of the multi-GPU path, with device-to-device
copies as the transport).  P-slab results must be BITWISE equal to the
1-slab run: every node's arithmetic and accumulation order is the same."""
import numpy as np
import pytest

from parity import assert_parity, group_errors
from paper_conf_sc_valero_laravgr23_b200 import distributed, inputs

pytestmark = pytest.mark.gpu

CASES = [
    ("D3Q19", "recursive", (23, 17, 29), {"z-": {"kind": "wall"}, "z+": {"kind": "moving_wall", "u": [0.05, 0, 0]},
                                          "y-": {"kind": "wall"}, "y+": {"kind": "wall"}}),
    ("D3Q27", "projective", (19, 13, 21), {}),  # periodic z: rank 0 <-> rank P-1
    ("D3Q19", "projective", (31, 19, 24), {"x-": {"kind": "velocity", "u": [0.04, 0, 0]},
                                           "x+": {"kind": "pressure", "rho": 1.0},
                                           "y-": {"kind": "wall"}, "y+": {"kind": "wall"},
                                           "z-": {"kind": "wall"}, "z+": {"kind": "wall"}}),
    ("D2Q9", "recursive", (70, 61, 1), {"x-": {"kind": "wall"}, "x+": {"kind": "wall"}, "y-": {"kind": "wall"},
                                        "y+": {"kind": "moving_wall", "u": [0.1, 0, 0]}}),
]


@pytest.mark.parametrize("P", [2, 3, 4])
@pytest.mark.parametrize("case", range(len(CASES)))
def test_slab_group_bitwise(case, P):
    from paper_conf_sc_valero_laravgr23_b200 import mrlbm
    lat, reg, (nx, ny, nz), b = CASES[case]
    D = 2 if lat == "D2Q9" else 3
    m0 = inputs.smooth_state(D, nx, ny, nz, U=0.05)
    steps = 37
    with mrlbm.Solver(lat, nx, ny, nz, 0.7, reg, b) as one:
        one.set_moments(m0)
        one.step(steps)
        ref = one.get_moments()
    slabs = [mrlbm.Solver(lat, nx, ny, nz, 0.7, reg, b, rank=r, nranks=P) for r in range(P)]
    try:
        for r, s in enumerate(slabs):
            s.set_moments(distributed.slab_of(m0, P, r))
        mrlbm.step_group(slabs, steps)
        got = np.concatenate([s.get_moments() for s in slabs], axis=1)
        with pytest.raises(mrlbm.MRLBMError):
            slabs[0].step(1)  # group handles refuse the single-handle path
    finally:
        for s in slabs:
            s.close()
    assert np.array_equal(got, ref), group_errors(got, ref, D)


def test_slab_group_vs_oracle():
    import oracle
    from paper_conf_sc_valero_laravgr23_b200 import mrlbm
    lat, reg, (nx, ny, nz), b = CASES[0]
    m0 = inputs.smooth_state(3, nx, ny, nz, U=0.05)
    o = oracle.Oracle(lat, nx, ny, nz, 0.7, reg, b)
    o.set_moments(m0)
    o.step(50)
    slabs = [mrlbm.Solver(lat, nx, ny, nz, 0.7, reg, b, rank=r, nranks=3) for r in range(3)]
    for r, s in enumerate(slabs):
        s.set_moments(distributed.slab_of(m0, 3, r))
    mrlbm.step_group(slabs, 50)
    got = np.concatenate([s.get_moments() for s in slabs], axis=1)
    for s in slabs:
        s.close()
    assert_parity(group_errors(got, o.get_moments(), 3), "fp64", "slab group vs oracle")
