"""Pins of the oracle's BGK collision (Alg. 1 lines 21-25; the
paper's standard-representation "ST" reference) against
facts that do not retype its formula: the tau = 1 textbook equilibrium,
conservation, the spectral picture of BGK (every non-equilibrium component,
hydrodynamic or ghost, is scaled by 1 - 1/tau, whereas the projective
regularization removes the ghosts), BGK == projective on a regularized input,
a brute-force np.roll stepper and the Taylor-Green viscosity."""
import math

import numpy as np
import pytest

from herm import CS2, moments, textbook_feq
from paper_conf_sc_valero_laravgr23_b200 import inputs

LATS = ["D2Q9", "D3Q19", "D3Q27"]


def random_f(oracle_mod, lat, rng, amp=1e-2):
    c, w, _, _ = oracle_mod.lattice_tables(lat)
    D = 2 if lat == "D2Q9" else 3
    u = np.zeros(3)
    u[:D] = rng.uniform(-0.1, 0.1, D)
    f = textbook_feq(c, w, rng.uniform(0.9, 1.1), u) + amp * w * rng.standard_normal(len(w))
    return c, w, f


@pytest.mark.parametrize("lat", LATS)
def test_bgk_tau_one_is_textbook_equilibrium(oracle_mod, lat):
    rng = np.random.default_rng(11)
    for _ in range(10):
        c, w, f = random_f(oracle_mod, lat, rng)
        rho, u, _ = moments(c, f)
        assert np.allclose(oracle_mod.collide_node(lat, "bgk", 1.0, f), textbook_feq(c, w, rho, u),
                           rtol=1e-14, atol=1e-16)


@pytest.mark.parametrize("lat", LATS)
def test_bgk_conserves_mass_momentum(oracle_mod, lat):
    rng = np.random.default_rng(12)
    for _ in range(10):
        c, w, f = random_f(oracle_mod, lat, rng)
        fs = oracle_mod.collide_node(lat, "bgk", rng.uniform(0.51, 2.0), f)
        assert math.isclose(fs.sum(), f.sum(), rel_tol=1e-14)
        assert np.allclose(c.T @ fs, c.T @ f, atol=1e-15)


def _hydro_basis(c, w, D):
    """w_i * {1, c, H2} sampled on the lattice: the span the projective
    regularization keeps (orders <= 2)."""
    cols = [np.ones(len(c))] + [c[:, a].astype(float) for a in range(D)]
    for a in range(D):
        for b in range(a, D):
            cols.append(c[:, a] * c[:, b] - (CS2 if a == b else 0.0))
    return (w[:, None] * np.array(cols).T)


@pytest.mark.parametrize("lat", LATS)
def test_bgk_scales_every_nonequilibrium_mode_projective_drops_ghosts(oracle_mod, lat):
    """Decompose f - f^eq (textbook) into the span of w*{1,c,H2} and its
    complement (least squares, independent of either collision).  BGK scales
    both parts by 1 - 1/tau; the projective operator keeps the first scaled and
    removes the complement (the 'ghost' / higher-order part)."""
    rng = np.random.default_rng(13)
    D = 2 if lat == "D2Q9" else 3
    for _ in range(5):
        c, w, f = random_f(oracle_mod, lat, rng)
        tau = rng.uniform(0.55, 1.8)
        rho, u, _ = moments(c, f)
        feq = textbook_feq(c, w, rho, u)
        B = _hydro_basis(c, w, D)
        coef, *_ = np.linalg.lstsq(B, f - feq, rcond=None)
        hydro = B @ coef
        ghost = (f - feq) - hydro
        assert np.abs(ghost).max() > 1e-5  # the random input has a ghost part
        fb = oracle_mod.collide_node(lat, "bgk", tau, f)
        assert np.allclose(fb, feq + (1 - 1 / tau) * (hydro + ghost), atol=1e-15)
        fp = oracle_mod.collide_node(lat, "projective", tau, f)
        # projective: f^eq plus the relaxed second-order part only.  The
        # least-squares 'hydro' part is the orthogonal projection in the plain
        # inner product, so compare the moments that define it instead
        _, _, Pb = moments(c, fb)
        _, _, Pp = moments(c, fp)
        assert np.allclose(Pb[:D, :D], Pp[:D, :D], atol=1e-15)
        assert not np.allclose(fb, fp, atol=1e-9)


@pytest.mark.parametrize("lat", LATS)
def test_bgk_equals_projective_on_regularized_input(oracle_mod, lat):
    """A regularized population (f^eq + second-order Hermite part, what
    set_moments builds) has no ghost component: BGK and projective agree."""
    rng = np.random.default_rng(14)
    D = 2 if lat == "D2Q9" else 3
    for _ in range(10):
        m = inputs.random_state(D, 1, 1, 1, U=0.1, seed=int(rng.integers(1 << 30)))
        o = oracle_mod.Oracle(lat, 1, 1, 1, 0.8, "bgk")
        o.set_moments(m.reshape(len(m), -1))
        f = o.get_f().reshape(-1)
        tau = rng.uniform(0.55, 1.8)
        assert np.allclose(oracle_mod.collide_node(lat, "bgk", tau, f),
                           oracle_mod.collide_node(lat, "projective", tau, f), atol=1e-15)


def _numpy_bgk_periodic(c, w, f, tau, steps):
    """Brute force: textbook BGK collide (Alg. 1), np.roll push streaming."""
    f = f.copy()
    D = 2 if np.all(c[:, 2] == 0) else 3
    for _ in range(steps):
        rho = f.sum(0)
        j = np.einsum("ia,i...->a...", c.astype(float), f)
        u = j / rho
        cu = np.einsum("ia,a...->i...", c.astype(float), u)
        usq = (u * u).sum(0)
        feq = w.reshape((-1,) + (1,) * (f.ndim - 1)) * rho * (1 + 3 * cu + 4.5 * cu * cu - 1.5 * usq)
        fs = f - (f - feq) / tau
        for i in range(len(c)):
            # array axes: 2D [y][x], 3D [z][y][x]
            shift = (int(c[i, 1]), int(c[i, 0])) if D == 2 else (int(c[i, 2]), int(c[i, 1]), int(c[i, 0]))
            f[i] = np.roll(fs[i], shift, axis=tuple(range(D)))
    return f


@pytest.mark.parametrize("lat", LATS)
def test_bgk_oracle_matches_roll_stepper(oracle_mod, lat):
    D = 2 if lat == "D2Q9" else 3
    nx, ny, nz = (13, 11, 1) if D == 2 else (7, 6, 5)
    c, w, _, _ = oracle_mod.lattice_tables(lat)
    o = oracle_mod.Oracle(lat, nx, ny, nz, 0.7, "bgk")
    o.set_moments(inputs.random_state(D, nx, ny, nz, U=0.05))
    f0 = o.get_f()
    # add a ghost-mode component so that BGK differs from the regularized runs
    rng = np.random.default_rng(15)
    f0 = f0 + 1e-3 * w.reshape((-1,) + (1,) * D) * rng.standard_normal(f0.shape)
    o.set_f(f0)
    o.step(40)
    ref = _numpy_bgk_periodic(c.astype(np.int64), w, f0, 0.7, 40)
    assert np.abs(o.get_f() - ref).max() < 1e-14


def test_bgk_taylor_green_viscosity(oracle_mod):
    """BGK's shear viscosity is nu = c_s^2 (tau - 1/2): TGV energy decays at 4 nu k^2."""
    n, steps, tau, U = 48, 400, 0.8, 0.01
    nu, k = (tau - 0.5) / 3, 2 * np.pi / n
    m = inputs.taylor_green_2d(n, U, tau)
    o = oracle_mod.Oracle("D2Q9", n, n, 1, tau, "bgk", threads=4)
    o.set_moments(m)
    e0 = (m[1] ** 2 + m[2] ** 2).sum()
    o.step(steps)
    mm = o.get_moments()
    rate = -np.log((mm[1] ** 2 + mm[2] ** 2).sum() / e0) / steps
    assert abs(rate / (4 * nu * k * k) - 1) < 0.01


@pytest.mark.parametrize("lat", LATS)
def test_bgk_closed_cavity_conserves_mass(oracle_mod, lat):
    D = 2 if lat == "D2Q9" else 3
    nx, ny, nz = (20, 16, 1) if D == 2 else (9, 8, 7)
    faces = ["x-", "x+", "y-", "y+"] + (["z-", "z+"] if D == 3 else [])
    b = {f: {"kind": "wall"} for f in faces}
    b["y+"] = {"kind": "moving_wall", "u": [0.08, 0.0, 0.0]}
    o = oracle_mod.Oracle(lat, nx, ny, nz, 0.65, "bgk", b)
    o.set_moments(inputs.perturbed_rest(D, nx, ny, nz, U=0.05))
    m0 = o.get_f().sum()
    o.step(300)
    assert abs(o.get_f().sum() - m0) / m0 < 1e-13
    assert o.get_moments()[1][..., -1, :].mean() > 0.008
