"""GPU parity of the distribution representation (ST, the paper's comparison
baseline: Alg. 1) against the CPU oracle,
through the same C ABI (representation = MRLBM_DISTRIBUTIONS).  Metric and
tolerances as the MR tests (1e-11 fp64, 1e-4 fp32)."""
import numpy as np
import pytest

from parity import THREADS, assert_parity, group_errors
from paper_conf_sc_valero_laravgr23_b200 import inputs

pytestmark = pytest.mark.gpu

LATS = ["D2Q9", "D3Q19", "D3Q27"]


def walls(D, lid=None):
    faces = ["x-", "x+", "y-", "y+"] + (["z-", "z+"] if D == 3 else [])
    b = {f: {"kind": "wall"} for f in faces}
    if lid:
        b[lid[0]] = {"kind": "moving_wall", "u": lid[1]}
    return b


def grid(lat):
    return (131, 67, 1) if lat == "D2Q9" else (37, 29, 23)


def ghost_populations(oracle_mod, lat, nx, ny, nz, m0, seed=5):
    """regularized populations of m0 plus a non-hydrodynamic (ghost) part, so
    that BGK differs from the regularized operators"""
    D = 2 if lat == "D2Q9" else 3
    o = oracle_mod.Oracle(lat, nx, ny, nz, 0.7, "bgk")
    o.set_moments(m0)
    f = o.get_f()
    _, w, _, _ = oracle_mod.lattice_tables(lat)
    rng = np.random.default_rng(seed)
    return f + 2e-4 * w.reshape((-1,) + (1,) * D) * rng.standard_normal(f.shape)


def run_st(oracle_mod, lat, coll, nx, ny, nz, tau, boundary, steps, precision="fp64", f0=None, m0=None):
    from paper_conf_sc_valero_laravgr23_b200 import mrlbm
    D = 2 if lat == "D2Q9" else 3
    o = oracle_mod.Oracle(lat, nx, ny, nz, tau, coll, boundary, threads=THREADS)
    with mrlbm.Solver(lat, nx, ny, nz, tau, coll, boundary, precision=precision, representation="distributions") as s:
        if f0 is not None:
            o.set_f(f0)
            s.set_populations(f0)
        else:
            o.set_moments(m0)
            s.set_moments(m0)
        o.step(steps)
        s.step(steps)
        got = s.get_moments()
        pops = s.get_populations()
        assert s.launch_count() == steps
    return group_errors(got, o.get_moments(), D), pops, o.get_populations()


@pytest.mark.parametrize("precision", ["fp64", "fp32"])
@pytest.mark.parametrize("coll", ["bgk", "projective", "recursive"])
@pytest.mark.parametrize("lat", LATS)
def test_st_periodic(oracle_mod, lat, coll, precision):
    nx, ny, nz = grid(lat)
    D = 2 if lat == "D2Q9" else 3
    m0 = inputs.smooth_state(D, nx, ny, nz, U=0.05)
    f0 = ghost_populations(oracle_mod, lat, nx, ny, nz, m0) if coll == "bgk" else None
    steps = 1000 if D == 2 else 200
    errs, pops, ref = run_st(oracle_mod, lat, coll, nx, ny, nz, 0.6, {}, steps, precision, f0=f0, m0=m0)
    assert_parity(errs, precision, f"ST {lat}-{coll} periodic")
    if precision == "fp64":
        assert np.abs(pops - ref).max() < 1e-13


@pytest.mark.parametrize("coll", ["bgk", "projective", "recursive"])
@pytest.mark.parametrize("lat", LATS)
def test_st_cavity_lid(oracle_mod, lat, coll):
    nx, ny, nz = grid(lat)
    D = 2 if lat == "D2Q9" else 3
    m0 = inputs.smooth_state(D, nx, ny, nz, U=0.05)
    b = walls(D, ("y+", [0.1, 0.0, 0.0]))
    if D == 3:
        b["z-"] = {"kind": "moving_wall", "u": [0.02, -0.03, 0.0]}
    steps = 1000 if D == 2 else 200
    errs, _, _ = run_st(oracle_mod, lat, coll, nx, ny, nz, 0.65, b, steps, m0=m0)
    assert_parity(errs, "fp64", f"ST {lat}-{coll} cavity")


@pytest.mark.parametrize("lat", LATS)
def test_st_mixed_faces_and_thin_shapes(oracle_mod, lat):
    D = 2 if lat == "D2Q9" else 3
    shapes = [(2, 2, 1), (129, 3, 1), (5, 200, 1)] if D == 2 else [(2, 2, 2), (130, 3, 4), (3, 5, 40)]
    for nx, ny, nz in shapes:
        b = {"y-": {"kind": "wall"}, "y+": {"kind": "moving_wall", "u": [0.05, 0, 0]}}
        m0 = inputs.smooth_state(D, nx, ny, nz, U=0.05)
        errs, _, _ = run_st(oracle_mod, lat, "bgk", nx, ny, nz, 0.7, b, 50, m0=m0)
        assert_parity(errs, "fp64", f"ST {lat} {nx}x{ny}x{nz}")


@pytest.mark.parametrize("lat", LATS)
def test_mr_and_st_agree_for_regularized_collisions(lat):
    """The paper's premise: MR is lossless, so MR and ST with
    the same regularized collision give the same trajectory (to rounding)."""
    from paper_conf_sc_valero_laravgr23_b200 import mrlbm
    nx, ny, nz = grid(lat)
    D = 2 if lat == "D2Q9" else 3
    m0 = inputs.smooth_state(D, nx, ny, nz, U=0.05)
    b = walls(D, ("y+", [0.1, 0.0, 0.0]))
    for reg in ("projective", "recursive"):
        out = []
        for rep in ("moments", "distributions"):
            with mrlbm.Solver(lat, nx, ny, nz, 0.65, reg, b, representation=rep) as s:
                s.set_moments(m0)
                s.step(300)
                out.append(s.get_moments())
        errs = group_errors(out[0], out[1], D)
        assert_parity(errs, "fp64", f"MR vs ST {lat}-{reg}")


@pytest.mark.parametrize("lat", LATS)
def test_mr_set_populations_stores_their_moments(oracle_mod, lat):
    from paper_conf_sc_valero_laravgr23_b200 import mrlbm
    nx, ny, nz = (19, 13, 1) if lat == "D2Q9" else (11, 9, 7)
    D = 2 if lat == "D2Q9" else 3
    m0 = inputs.smooth_state(D, nx, ny, nz, U=0.05)
    f0 = ghost_populations(oracle_mod, lat, nx, ny, nz, m0)
    o = oracle_mod.Oracle(lat, nx, ny, nz, 0.7, "recursive")
    o.set_f(f0)
    with mrlbm.Solver(lat, nx, ny, nz, 0.7, "recursive") as s:
        s.set_populations(f0)
        # moments of arbitrary populations: Q-term sums of O(1) values taken in
        # the shifted representation f - w (R16) on the GPU and unshifted in
        # the oracle, so the rounding floor is absolute, a few ulp(1); bound
        # 64 ulp(1) = 1.4e-14 on every moment (a wrong index or weight is >1e-4)
        assert np.abs(s.get_moments() - o.get_moments()).max() <= 64 * np.finfo(np.float64).eps
        o.step(20)
        s.step(20)
        assert_parity(group_errors(s.get_moments(), o.get_moments(), D), "fp64", "MR from populations")
