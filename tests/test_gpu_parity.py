"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle,
element by element on the same seeded inputs (SURVEY 8(c) metric and
BASELINE.json tolerances: 1e-11 fp64 / 1e-4 fp32 vs the fp64 oracle)."""
import numpy as np
import pytest

from parity import assert_parity, run_pair
from paper_conf_sc_valero_laravgr23_b200 import configs, inputs

pytestmark = pytest.mark.gpu

VARIANTS = [(l, r) for l in ("D2Q9", "D3Q19", "D3Q27") for r in ("projective", "recursive")]


def walls(D, lid=None):
    faces = ["x-", "x+", "y-", "y+"] + (["z-", "z+"] if D == 3 else [])
    b = {f: {"kind": "wall"} for f in faces}
    if lid:
        b[lid[0]] = {"kind": "moving_wall", "u": lid[1]}
    return b


def grid(lat, big=False):
    if lat == "D2Q9":
        return (131, 67, 1) if not big else (263, 131, 1)
    return (37, 29, 23)


@pytest.mark.parametrize("precision", ["fp64", "fp32"])
@pytest.mark.parametrize("lat,reg", VARIANTS)
def test_periodic_random(lat, reg, precision):
    nx, ny, nz = grid(lat)
    D = 2 if lat == "D2Q9" else 3
    m0 = inputs.smooth_state(D, nx, ny, nz, U=0.05)
    steps = 1000 if D == 2 else 200
    errs, _, _ = run_pair(lat, reg, nx, ny, nz, 0.6, {}, m0, steps, precision)
    assert_parity(errs, precision, f"{lat}-{reg} periodic")


@pytest.mark.parametrize("precision", ["fp64", "fp32"])
@pytest.mark.parametrize("lat,reg", VARIANTS)
def test_cavity_walls_and_lid(lat, reg, precision):
    nx, ny, nz = grid(lat)
    D = 2 if lat == "D2Q9" else 3
    m0 = inputs.smooth_state(D, nx, ny, nz, U=0.05)
    b = walls(D, ("y+", [0.1, 0.0, 0.0]))
    steps = 1000 if D == 2 else 200
    errs, got, _ = run_pair(lat, reg, nx, ny, nz, 0.65, b, m0, steps, precision)
    assert_parity(errs, precision, f"{lat}-{reg} cavity")


@pytest.mark.parametrize("lat,reg", VARIANTS)
def test_mixed_faces(lat, reg):
    """Periodic x, walls y, moving walls on the marching axis (3D z / 2D y)."""
    nx, ny, nz = (70, 33, 1) if lat == "D2Q9" else (33, 20, 17)
    D = 2 if lat == "D2Q9" else 3
    b = {"y-": {"kind": "wall"}, "y+": {"kind": "moving_wall", "u": [0.05, 0, 0.02 if D == 3 else 0]}}
    if D == 3:
        b = {"y-": {"kind": "wall"}, "y+": {"kind": "wall"},
             "z-": {"kind": "moving_wall", "u": [0.03, -0.02, 0]}, "z+": {"kind": "moving_wall", "u": [0.0, 0.04, 0]}}
    m0 = inputs.random_state(D, nx, ny, nz, U=0.05, seed=7)
    errs, _, _ = run_pair(lat, reg, nx, ny, nz, 0.7, b, m0, 100)
    assert_parity(errs, "fp64", f"{lat}-{reg} mixed")


@pytest.mark.parametrize("reg", ["projective", "recursive"])
@pytest.mark.parametrize("precision", ["fp64", "fp32"])
def test_c1_poiseuille_channel(reg, precision):
    """BASELINE configs[0] (C1): D2Q9 Poiseuille 128x64, velocity inlet,
    pressure outlet, walls; 1000 steps vs the oracle."""
    c = configs.c1()
    c.regularization = reg
    errs, got, _ = run_pair(c.lattice, reg, c.nx, c.ny, 1, c.tau, c.boundary, c.initial_moments(), 1000, precision)
    assert_parity(errs, precision, f"C1 {reg}")
    prof = inputs.poiseuille_profile(c.ny, c.U)
    assert np.abs(got[1] - prof[:, None]).max() / c.U < 5e-3


@pytest.mark.parametrize("lat,reg", [(l, r) for l in ("D3Q19", "D3Q27") for r in ("projective", "recursive")])
@pytest.mark.parametrize("axis", ["x", "y"])
def test_open_faces_3d(lat, reg, axis):
    """Velocity inlet + pressure outlet on the x (A) or y (B) faces, walls on
    the others (C5 shape, small)."""
    nx, ny, nz = 31, 19, 13
    U = 0.04
    if axis == "x":
        prof = inputs.channel3d_profile(ny, nz, U)
        b = {"x-": {"kind": "velocity", "u_profile": prof}, "x+": {"kind": "pressure", "rho": 1.0},
             "y-": {"kind": "wall"}, "y+": {"kind": "wall"}, "z-": {"kind": "wall"}, "z+": {"kind": "wall"}}
    else:
        b = {"y-": {"kind": "velocity", "u": [0.0, U, 0.0]}, "y+": {"kind": "pressure", "rho": 0.999},
             "x-": {"kind": "wall"}, "x+": {"kind": "moving_wall", "u": [0.0, 0.0, 0.01]}}
    m0 = inputs.smooth_state(3, nx, ny, nz, U=U)
    errs, _, _ = run_pair(lat, reg, nx, ny, nz, 0.62, b, m0, 150)
    assert_parity(errs, "fp64", f"{lat}-{reg} open {axis}")


@pytest.mark.parametrize("lat,reg", VARIANTS)
def test_populations(lat, reg):
    """mrlbm_get_populations = the oracle's post-collision f* (R17)."""
    import oracle
    from paper_conf_sc_valero_laravgr23_b200 import mrlbm
    nx, ny, nz = (17, 9, 1) if lat == "D2Q9" else (9, 7, 5)
    D = 2 if lat == "D2Q9" else 3
    m0 = inputs.random_state(D, nx, ny, nz)
    o = oracle.Oracle(lat, nx, ny, nz, 0.77, reg)
    o.set_moments(m0)
    ref = o.get_populations()
    with mrlbm.Solver(lat, nx, ny, nz, 0.77, reg) as s:
        s.set_moments(m0)
        got = s.get_populations()
    assert np.abs(got - ref).max() < 1e-14


@pytest.mark.parametrize("lat", ["D2Q9", "D3Q19"])
@pytest.mark.parametrize("shape", ["tiny", "one_tile", "tile_plus_one", "thin"])
def test_edge_shapes(lat, shape):
    """Degenerate and ragged extents around the tile sizes (2D tiles are 126
    nodes wide, 3D tiles 30 x 6)."""
    D = 2 if lat == "D2Q9" else 3
    shapes2 = {"tiny": (2, 2, 1), "one_tile": (126, 5, 1), "tile_plus_one": (127, 9, 1), "thin": (300, 2, 1)}
    shapes3 = {"tiny": (2, 2, 2), "one_tile": (30, 6, 4), "tile_plus_one": (31, 7, 3), "thin": (61, 2, 9)}
    nx, ny, nz = (shapes2 if D == 2 else shapes3)[shape]
    for b in ({}, walls(D, ("y+", [0.05, 0, 0]))):
        m0 = inputs.random_state(D, nx, ny, nz, U=0.05, seed=3)
        errs, _, _ = run_pair(lat, "recursive", nx, ny, nz, 0.8, b, m0, 50)
        assert_parity(errs, "fp64", f"{lat} {shape}")


@pytest.mark.parametrize("lat", ["D2Q9", "D3Q27"])
@pytest.mark.parametrize("precision", ["fp64", "fp32"])
def test_set_get_roundtrip(lat, precision):
    from paper_conf_sc_valero_laravgr23_b200 import mrlbm
    D = 2 if lat == "D2Q9" else 3
    nx, ny, nz = 45, 13, 7
    m0 = inputs.random_state(D, nx, ny, nz)
    with mrlbm.Solver(lat, nx, ny, nz, 0.7, "projective", precision=precision) as s:
        s.set_moments(m0)
        got = s.get_moments()
        s.step(0)
        assert s.launch_count() == 0
    if precision == "fp64":
        assert np.array_equal(got, m0)
    else:
        assert np.allclose(got, m0, rtol=1e-6, atol=1e-7)


def fast_ctas(cfg, nA, nC):
    """CTAs that take the boundary-free body (mrlbm_step_kernel: window
    inside the domain along A, segment holding neither the first nor the
    last layer along C) -- 2D only."""
    TA, L = cfg["TA"], cfg["seg_len"]
    tiles = [-1 + i * (TA - 2) for i in range(cfg["grid_x"])]
    nA_fast = sum(1 for a0 in tiles if a0 >= 0 and a0 + TA <= nA)
    segs = [(s * L, min(nC, (s + 1) * L) - 1) for s in range(cfg["grid_y"])]
    return nA_fast * sum(1 for c0, c1 in segs if c0 > 0 and c1 < nC - 1)


@pytest.mark.parametrize("precision", ["fp64", "fp32"])
@pytest.mark.parametrize("reg", ["projective", "recursive"])
@pytest.mark.parametrize("bc", ["periodic", "cavity"])
def test_interior_fast_body(bc, reg, precision):
    """A D2Q9 grid wide and tall enough that interior CTAs take the
    boundary-free body (4 tiles along x, several segments along y), next to
    boundary CTAs of every kind; element-by-element vs the oracle."""
    from paper_conf_sc_valero_laravgr23_b200 import mrlbm
    nx, ny = 400, 120
    m0 = inputs.smooth_state(2, nx, ny, 1, U=0.05)
    b = {} if bc == "periodic" else walls(2, ("y+", [0.1, 0.0, 0.0]))
    with mrlbm.Solver("D2Q9", nx, ny, 1, 0.6, reg, b, precision=precision) as s:
        cfg = s.kernel_config()
    assert fast_ctas(cfg, nx, ny) > 0, cfg
    errs, _, _ = run_pair("D2Q9", reg, nx, ny, 1, 0.6, b, m0, 500, precision)
    assert_parity(errs, precision, f"D2Q9-{reg} {bc} interior body")


@pytest.mark.parametrize("precision", ["fp64", "fp32"])
def test_device_io_roundtrip(precision):
    """set/get through device pointers (torch tensors produced on torch's
    current stream): same trajectory, bit for bit, as the host path."""
    import torch
    from paper_conf_sc_valero_laravgr23_b200 import mrlbm
    nx, ny, nz = 37, 29, 23
    m0 = inputs.smooth_state(3, nx, ny, nz, U=0.05)
    b = walls(3, ("y+", [0.05, 0.0, 0.0]))
    with mrlbm.Solver("D3Q19", nx, ny, nz, 0.7, "recursive", b, precision=precision) as s:
        s.set_moments(m0)
        s.step(40)
        ref = s.get_moments()
    dev = torch.device("cuda", 0)
    t_in = torch.from_numpy(m0).to(dev) * 1.0 + 0.0   # produced by kernels on torch's stream
    t_out = torch.full_like(t_in, float("nan"))
    with mrlbm.Solver("D3Q19", nx, ny, nz, 0.7, "recursive", b, precision=precision) as s:
        s.set_moments(t_in)
        del t_in                                      # the library copied it before returning
        s.step(40)
        s.get_moments_device(t_out)
    got = t_out.cpu().numpy()
    assert np.array_equal(got, ref)
