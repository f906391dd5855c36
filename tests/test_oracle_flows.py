"""Flow-level pins of the oracle: invariants, analytic solutions and an
independent moment-form stepper (SURVEY 8(c) pins 3, 4, 7, 8, 9, 10)."""
import numpy as np
import pytest

import mr_numpy
from paper_conf_sc_valero_laravgr23_b200 import inputs

VARIANTS = [(l, r) for l in ("D2Q9", "D3Q19", "D3Q27") for r in ("projective", "recursive")]


def small_grid(lat):
    return (24, 20, 1) if lat == "D2Q9" else (10, 9, 8)


def walls(D, lid=None, U=0.05):
    faces = ["x-", "x+", "y-", "y+"] + (["z-", "z+"] if D == 3 else [])
    b = {f: {"kind": "wall"} for f in faces}
    if lid:
        b[lid[0]] = {"kind": "moving_wall", "u": lid[1]}
    return b


@pytest.mark.parametrize("lat,reg", VARIANTS)
def test_periodic_conservation(oracle_mod, lat, reg):
    """Fully periodic: total mass and momentum are invariants (1000 steps in 2D)."""
    nx, ny, nz = small_grid(lat)
    D = 2 if lat == "D2Q9" else 3
    m0 = inputs.random_state(D, nx, ny, nz, U=0.05)
    o = oracle_mod.Oracle(lat, nx, ny, nz, 0.7, reg)
    o.set_moments(m0)
    f0 = o.get_f()
    c, _, _, _ = oracle_mod.lattice_tables(lat)
    mass0 = f0.sum()
    mom0 = np.einsum("ia,i...->a...", c.astype(float), f0).reshape(3, -1).sum(1)
    o.step(1000 if D == 2 else 100)
    f1 = o.get_f()
    assert abs(f1.sum() - mass0) / mass0 < 1e-13
    mom1 = np.einsum("ia,i...->a...", c.astype(float), f1).reshape(3, -1).sum(1)
    assert np.allclose(mom1, mom0, atol=1e-13 * mass0)


@pytest.mark.parametrize("lat,reg", VARIANTS)
def test_closed_cavity_mass_conservation(oracle_mod, lat, reg):
    """Walls on every face plus a moving lid (R13): mass is exactly conserved,
    including the lid links that also cross a side wall."""
    nx, ny, nz = small_grid(lat)
    D = 2 if lat == "D2Q9" else 3
    lids = [("y+", [0.08, 0.0, 0.0])] + ([("z-", [0.03, -0.05, 0.0])] if D == 3 else [])
    for lid in lids:
        o = oracle_mod.Oracle(lat, nx, ny, nz, 0.65, reg, walls(D, lid))
        o.set_moments(inputs.perturbed_rest(D, nx, ny, nz, U=0.05))
        m0 = o.get_f().sum()
        o.step(300)
        mm = o.get_moments()
        assert abs(o.get_f().sum() - m0) / m0 < 1e-13
        # the lid drives the flow in its own direction next to it
        if lid[0] == "y+":
            assert mm[1][..., -1, :].mean() > 0.1 * lid[1][0]


@pytest.mark.parametrize("lat,reg", VARIANTS)
def test_moment_form_stepper_equivalence(oracle_mod, lat, reg):
    """Lossless moment representation: an independent
    numpy moment-form stepper (pull streaming, closed-form recursion) and the
    distribution-form oracle give the same moments."""
    nx, ny, nz = (7, 6, 1) if lat == "D2Q9" else (5, 4, 6)
    D = 2 if lat == "D2Q9" else 3
    tabs = oracle_mod.lattice_tables(lat)
    cases = [{}, walls(D, ("y+", [0.07, 0.0, 0.0]))]
    if D == 3:
        cases.append({"z-": {"kind": "wall"}, "z+": {"kind": "moving_wall", "u": [0.02, 0.04, 0.0]},
                      "x-": {"kind": "wall"}, "x+": {"kind": "wall"}})
    for b in cases:
        m = inputs.random_state(D, nx, ny, nz, U=0.08, seed=5)
        o = oracle_mod.Oracle(lat, nx, ny, nz, 0.62, reg, b)
        o.set_moments(m)
        for _ in range(6):
            m = mr_numpy.step(m, tabs, reg, 0.62, b, D)
        o.step(6)
        got = o.get_moments()
        assert np.allclose(got, m, rtol=0, atol=2e-15), np.abs(got - m).max()


def _poiseuille_error(oracle_mod, lat, reg, ny, steps, from_rest=False, nx=None, tau=0.8, U=0.05):
    nx = nx or 2 * ny
    prof = inputs.poiseuille_profile(ny, U)
    if lat == "D2Q9":
        up = np.stack([prof, 0 * prof], 1)
        b = {"x-": {"kind": "velocity", "u_profile": up}, "x+": {"kind": "pressure", "rho": 1.0},
             "y-": {"kind": "wall"}, "y+": {"kind": "wall"}}
        m = inputs.poiseuille_state(nx, ny, U, tau)
        if from_rest:
            m = inputs.perturbed_rest(2, nx, ny, 1, U=0.0, pi_neq=False)
        o = oracle_mod.Oracle(lat, nx, ny, 1, tau, reg, b, threads=4)
    else:
        nz = 3  # periodic z: plane Poiseuille in a 3D lattice
        up = np.zeros((nz, ny, 3))
        up[..., 0] = prof[None, :]
        b = {"x-": {"kind": "velocity", "u_profile": up}, "x+": {"kind": "pressure", "rho": 1.0},
             "y-": {"kind": "wall"}, "y+": {"kind": "wall"}}
        m2 = inputs.poiseuille_state(nx, ny, U, tau)
        z = np.zeros((nz, ny, nx))
        rho, ux, uy, pxx, pyy, pxy = [np.broadcast_to(a, (nz, ny, nx)) for a in m2]
        m = np.stack([rho, ux, uy, z, pxx, pyy, z, pxy, z, z])
        o = oracle_mod.Oracle(lat, nx, ny, nz, tau, reg, b, threads=4)
    o.set_moments(m)
    o.step(steps)
    mm = o.get_moments()
    ux = mm[1]
    return np.abs(ux - prof[:, None]).max() / U, mm


@pytest.mark.parametrize("reg", ["projective", "recursive"])
def test_poiseuille_channel_d2q9(oracle_mod, reg):
    """Pin 7 (C1 shape): velocity inlet + pressure outlet + halfway walls keep
    the analytic Poiseuille state within 5e-3 U after 1000 steps at H=64 and
    converge at (near) second order."""
    e16, _ = _poiseuille_error(oracle_mod, "D2Q9", reg, 16, 1000)
    e32, _ = _poiseuille_error(oracle_mod, "D2Q9", reg, 32, 1000)
    e64, mm = _poiseuille_error(oracle_mod, "D2Q9", reg, 64, 1000)
    assert e64 < 5e-3
    assert e16 / e32 > 2.0 and e32 / e64 > 2.5
    # mirror symmetry about the channel axis (pin 10): u_x even, u_y odd
    assert np.allclose(mm[1], mm[1][::-1], atol=1e-13)
    assert np.allclose(mm[2], -mm[2][::-1], atol=1e-13)


def test_poiseuille_develops_from_rest(oracle_mod):
    """Started from rest, the channel converges to the analytic profile."""
    e, mm = _poiseuille_error(oracle_mod, "D2Q9", "projective", 16, 8000, from_rest=True, nx=32, tau=0.9)
    assert e < 3e-2
    # outlet density is the prescribed one
    assert np.allclose(mm[0][:, -1], 1.0, atol=1e-12)


@pytest.mark.parametrize("lat", ["D3Q19", "D3Q27"])
@pytest.mark.parametrize("reg", ["projective", "recursive"])
def test_poiseuille_channel_3d(oracle_mod, lat, reg):
    e32, mm = _poiseuille_error(oracle_mod, lat, reg, 32, 400)
    e16, _ = _poiseuille_error(oracle_mod, lat, reg, 16, 400)
    assert e32 < 8e-3 and e16 / e32 > 2.0
    assert np.abs(mm[3]).max() < 1e-13  # no z-velocity develops
    assert np.allclose(mm[1], mm[1][:, ::-1], atol=1e-13)


@pytest.mark.parametrize("reg", ["projective", "recursive"])
def test_taylor_green_2d_decay(oracle_mod, reg):
    """Pin 8: kinetic energy decays at 4 nu k^2 with nu = c_s^2 (tau - 1/2)."""
    errs = []
    for n, steps in ((32, 300), (64, 600)):
        tau, U = 0.8, 0.01
        nu, k = (tau - 0.5) / 3, 2 * np.pi / n
        m = inputs.taylor_green_2d(n, U, tau)
        o = oracle_mod.Oracle("D2Q9", n, n, 1, tau, reg, threads=4)
        o.set_moments(m)
        e0 = (m[1] ** 2 + m[2] ** 2).sum()
        o.step(steps)
        mm = o.get_moments()
        rate = -np.log((mm[1] ** 2 + mm[2] ** 2).sum() / e0) / steps
        errs.append(abs(rate / (4 * nu * k * k) - 1))
        # velocity field keeps its analytic shape
        ma = inputs.taylor_green_2d(n, U, tau, t=steps)
        assert np.abs(mm[1] - ma[1]).max() < 0.02 * np.abs(ma[1]).max()
    assert errs[0] < 0.01 and errs[1] < errs[0]


@pytest.mark.parametrize("lat", ["D3Q19", "D3Q27"])
@pytest.mark.parametrize("axis", [0, 1, 2])
def test_taylor_green_3d_extruded_decay(oracle_mod, lat, axis):
    tau, U, n = 0.8, 0.01, 24
    nu, k = (tau - 0.5) / 3, 2 * np.pi / n
    m = inputs.taylor_green_3d_extruded(n, 3, U, tau, axis)
    ext = [n, n, n]
    ext[axis] = 3
    o = oracle_mod.Oracle(lat, *ext, tau, "recursive", threads=4)
    o.set_moments(m)
    e0 = (m[1:4] ** 2).sum()
    o.step(150)
    mm = o.get_moments()
    rate = -np.log((mm[1:4] ** 2).sum() / e0) / 150
    assert abs(rate / (4 * nu * k * k) - 1) < 0.01
    assert np.abs(mm[1 + axis]).max() < 1e-14  # no velocity along the extrusion axis


@pytest.mark.parametrize("lat,reg", VARIANTS)
def test_initialization_independence(oracle_mod, lat, reg):
    """Pin 9: two initial populations with the same (rho, u, Pi) give the same
    trajectory (collision reads only rho, u, Pi^neq)."""
    nx, ny, nz = small_grid(lat)
    D = 2 if lat == "D2Q9" else 3
    b = walls(D, ("y+", [0.05, 0, 0]))
    m = inputs.perturbed_rest(D, nx, ny, nz)
    a = oracle_mod.Oracle(lat, nx, ny, nz, 0.7, reg, b)
    a.set_moments(m)
    f = a.get_f()
    c, w, _, _ = oracle_mod.lattice_tables(lat)
    # a ghost field orthogonal to 1, c_a and c_a c_b (zero rho, j, Pi)
    basis = [np.ones(len(w))] + [c[:, p].astype(float) for p in range(D)]
    basis += [(c[:, p] * c[:, q]).astype(float) for p in range(D) for q in range(p, D)]
    B = np.array(basis).T
    rng = np.random.default_rng(3)
    g = rng.standard_normal((len(w),) + f.shape[1:])
    coef = np.linalg.lstsq(B, g.reshape(len(w), -1), rcond=None)[0]
    g = g - (B @ coef).reshape(g.shape)
    bo = oracle_mod.Oracle(lat, nx, ny, nz, 0.7, reg, b)
    bo.set_f(f + 1e-3 * g)
    assert np.allclose(bo.get_moments(), m, atol=1e-15)
    a.step(20)
    bo.step(20)
    assert np.allclose(a.get_moments(), bo.get_moments(), atol=1e-14)


@pytest.mark.parametrize("lat", ["D2Q9", "D3Q19", "D3Q27"])
def test_mirror_symmetry_closed_box(oracle_mod, lat):
    """Pin 10: a state mirror-symmetric in x inside a closed box stays symmetric."""
    nx, ny, nz = small_grid(lat)
    D = 2 if lat == "D2Q9" else 3
    m = inputs.perturbed_rest(D, nx, ny, nz, U=0.05)
    flip = lambda a: a[..., ::-1]
    # symmetrize: rho, u_y, u_z, diagonal Pi, Pi_yz even in x; u_x, Pi_xy, Pi_xz odd
    odd = {1, 5} if D == 2 else {1, 7, 8}
    ms = np.array([0.5 * (m[k] - flip(m[k])) if k in odd else 0.5 * (m[k] + flip(m[k])) for k in range(len(m))])
    ms[0] += 1.0 - ms[0].mean()
    for reg in ("projective", "recursive"):
        o = oracle_mod.Oracle(lat, nx, ny, nz, 0.7, reg, walls(D))
        o.set_moments(ms)
        o.step(100)
        mm = o.get_moments()
        for k in range(len(mm)):
            s = -1 if k in odd else 1
            assert np.allclose(mm[k], s * flip(mm[k]), atol=1e-14)
