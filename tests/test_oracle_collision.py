"""Node-level pins of the oracle's collision operators (eqs 4, 8-14) against
closed forms that do not share the oracle's formulas."""
import math

import numpy as np
import pytest

from herm import (CS2, d1q3_product, he, idx_of, moments, projective_moment_form,
                  recursive_moment_form, textbook_feq, aneq_pairsum)

LATS = ["D2Q9", "D3Q19", "D3Q27"]
REGS = ["projective", "recursive"]


def random_f(oracle_mod, lat, rng, zero_u=False):
    c, w, _, _ = oracle_mod.lattice_tables(lat)
    D = 2 if lat == "D2Q9" else 3
    rho = rng.uniform(0.9, 1.1)
    u = np.zeros(3)
    if not zero_u:
        u[:D] = rng.uniform(-0.1, 0.1, D)
    f = textbook_feq(c, w, rho, u) + 1e-3 * w * rng.standard_normal(len(w))
    return c, w, f


@pytest.mark.parametrize("lat", LATS)
def test_feq_is_textbook_bgk_equilibrium(oracle_mod, lat):
    rng = np.random.default_rng(1)
    c, w, _, _ = oracle_mod.lattice_tables(lat)
    D = 2 if lat == "D2Q9" else 3
    for _ in range(20):
        rho = rng.uniform(0.5, 1.5)
        u = np.zeros(3)
        u[:D] = rng.uniform(-0.2, 0.2, D)
        assert np.allclose(oracle_mod.feq(lat, rho, u[:D]), textbook_feq(c, w, rho, u), rtol=1e-14, atol=1e-16)
        # moments of f^eq: rho, rho u, Pi^eq = rho u u
        r, uu, Pi = moments(c, oracle_mod.feq(lat, rho, u[:D]))
        assert math.isclose(r, rho, rel_tol=1e-14)
        assert np.allclose(uu, u, atol=1e-15)
        assert np.allclose(Pi[:D, :D], rho * np.outer(u, u)[:D, :D], atol=1e-15)


@pytest.mark.parametrize("lat", LATS)
@pytest.mark.parametrize("reg", REGS)
def test_collision_conserves_mass_momentum(oracle_mod, lat, reg):
    rng = np.random.default_rng(2)
    for _ in range(20):
        c, w, f = random_f(oracle_mod, lat, rng)
        fs = oracle_mod.collide_node(lat, reg, rng.uniform(0.51, 2.0), f)
        assert math.isclose(fs.sum(), f.sum(), rel_tol=1e-14)
        assert np.allclose(c.T @ fs, c.T @ f, atol=1e-15)


@pytest.mark.parametrize("lat,reg", [(l, r) for l in LATS for r in REGS if (l, r) != ("D3Q19", "recursive")])
def test_second_moment_relaxes_per_eq10(oracle_mod, lat, reg):
    rng = np.random.default_rng(3)
    D = 2 if lat == "D2Q9" else 3
    for _ in range(20):
        c, w, f = random_f(oracle_mod, lat, rng)
        tau = rng.uniform(0.51, 2.0)
        rho, u, Pi = moments(c, f)
        Pneq = Pi - rho * np.outer(u, u)
        fs = oracle_mod.collide_node(lat, reg, tau, f)
        _, _, Pis = moments(c, fs)
        expect = rho * np.outer(u, u) + (1 - 1 / tau) * Pneq
        assert np.allclose(Pis[:D, :D], expect[:D, :D], atol=1e-15)


def test_d3q19_recursive_second_moment_offset(oracle_mod):
    """R11: with the literal eq-14 basis, Pi_aa(f*) = Pi*_aa - 3/4 a*_{bbgg}
    (b,g the other two axes); off-diagonals exact."""
    rng = np.random.default_rng(4)
    c, w, _, h = oracle_mod.lattice_tables("D3Q19")
    for _ in range(10):
        _, _, f = random_f(oracle_mod, "D3Q19", rng)
        tau = rng.uniform(0.51, 2.0)
        rho, u, Pi = moments(c, f)
        Pneq = Pi - rho * np.outer(u, u)
        A, _ = recursive_moment_form(c, w, h, tau, rho, u, Pneq)
        fs = oracle_mod.collide_node("D3Q19", "recursive", tau, f)
        _, _, Pis = moments(c, fs)
        Pstar = rho * np.outer(u, u) + (1 - 1 / tau) * Pneq
        for a in range(3):
            others = [b for b in range(3) if b != a]
            hh = [0, 0, 0]
            for b in others:
                hh[b] = 2
            assert math.isclose(Pis[a, a], Pstar[a, a] - 0.75 * A[tuple(hh)], abs_tol=1e-15)
        for a, b in [(0, 1), (0, 2), (1, 2)]:
            assert math.isclose(Pis[a, b], Pstar[a, b], abs_tol=1e-15)


@pytest.mark.parametrize("lat", LATS)
def test_projective_tau1_is_equilibrium(oracle_mod, lat):
    rng = np.random.default_rng(5)
    for _ in range(10):
        c, w, f = random_f(oracle_mod, lat, rng)
        rho, u, _ = moments(c, f)
        fs = oracle_mod.collide_node(lat, "projective", 1.0, f)
        assert np.allclose(fs, textbook_feq(c, w, rho, u), atol=1e-15)


@pytest.mark.parametrize("lat", ["D2Q9", "D3Q27"])
def test_recursive_tau1_is_d1q3_product_equilibrium(oracle_mod, lat):
    rng = np.random.default_rng(6)
    for _ in range(10):
        c, w, f = random_f(oracle_mod, lat, rng)
        rho, u, _ = moments(c, f)
        fs = oracle_mod.collide_node(lat, "recursive", 1.0, f)
        assert np.allclose(fs, d1q3_product(c, rho, u, 2 if lat == "D2Q9" else 3), atol=1e-15)


@pytest.mark.parametrize("lat", LATS)
def test_recursive_equals_projective_at_rest(oracle_mod, lat):
    rng = np.random.default_rng(7)
    for _ in range(10):
        c, w, f = random_f(oracle_mod, lat, rng, zero_u=True)
        # symmetric populations: zero momentum up to summation rounding
        _, _, opp, _ = oracle_mod.lattice_tables(lat)
        f = 0.5 * (f + f[opp])
        assert np.allclose(c.T @ f, 0, atol=1e-16)
        tau = rng.uniform(0.51, 2.0)
        fp = oracle_mod.collide_node(lat, "projective", tau, f)
        fr = oracle_mod.collide_node(lat, "recursive", tau, f)
        assert np.allclose(fp, fr, atol=1e-16)


@pytest.mark.parametrize("lat", LATS)
def test_eq9_distribution_form_equals_eq10_11_moment_form(oracle_mod, lat):
    """P:L103 'equivalently formulated in moment space': the oracle's eq 9
    must equal eqs 10-11 written out independently."""
    rng = np.random.default_rng(8)
    for _ in range(20):
        c, w, f = random_f(oracle_mod, lat, rng)
        tau = rng.uniform(0.51, 2.0)
        rho, u, Pi = moments(c, f)
        Pneq = Pi - rho * np.outer(u, u)
        expect = projective_moment_form(c, w, tau, rho, u, Pneq)
        assert np.allclose(oracle_mod.collide_node(lat, "projective", tau, f), expect, atol=2e-16)


@pytest.mark.parametrize("lat", LATS)
def test_recursive_matches_pairsum_closed_form(oracle_mod, lat):
    rng = np.random.default_rng(9)
    c, w, _, h = oracle_mod.lattice_tables(lat)
    for _ in range(20):
        _, _, f = random_f(oracle_mod, lat, rng)
        tau = rng.uniform(0.51, 2.0)
        rho, u, Pi = moments(c, f)
        Pneq = Pi - rho * np.outer(u, u)
        _, expect = recursive_moment_form(c, w, h, tau, rho, u, Pneq)
        assert np.allclose(oracle_mod.collide_node(lat, "recursive", tau, f), expect, atol=2e-16)


@pytest.mark.parametrize("lat", ["D2Q9", "D3Q27"])
def test_recursive_reconstruction_projects_back(oracle_mod, lat):
    """On orthogonal bases the Hermite projections of f* return every
    collided coefficient: sum_i He_h(c_i) f*_i = A*_h (eq 14 inverted)."""
    rng = np.random.default_rng(10)
    c, w, _, h = oracle_mod.lattice_tables(lat)
    for _ in range(10):
        _, _, f = random_f(oracle_mod, lat, rng)
        tau = rng.uniform(0.51, 2.0)
        rho, u, Pi = moments(c, f)
        Pneq = Pi - rho * np.outer(u, u)
        A, _ = recursive_moment_form(c, w, h, tau, rho, u, Pneq)
        fs = oracle_mod.collide_node(lat, "recursive", tau, f)
        for hh, a in A.items():
            assert math.isclose(np.sum(he(hh, c) * fs), a, abs_tol=2e-16)


def test_recursion_closed_forms(oracle_mod):
    """SURVEY App. A named closed forms of the recursion, orders 3-6, and
    symmetry of the recursion under index permutation."""
    rng = np.random.default_rng(11)
    x, y, z = 0, 1, 2
    for _ in range(20):
        u = rng.uniform(-0.2, 0.2, 3)
        P = rng.standard_normal((3, 3))
        P = P + P.T
        a = lambda idx: oracle_mod.aneq(idx, u, P)
        assert math.isclose(a([x, x, y]), 2 * u[x] * P[x, y] + u[y] * P[x, x], abs_tol=1e-15)
        assert math.isclose(a([x, y, z]), u[x] * P[y, z] + u[y] * P[x, z] + u[z] * P[x, y], abs_tol=1e-15)
        assert math.isclose(a([x, x, y, y]), u[y] ** 2 * P[x, x] + u[x] ** 2 * P[y, y] + 4 * u[x] * u[y] * P[x, y],
                            abs_tol=1e-15)
        assert math.isclose(a([x, x, y, z]), u[y] * u[z] * P[x, x] + 2 * u[x] * u[z] * P[x, y]
                            + 2 * u[x] * u[y] * P[x, z] + u[x] ** 2 * P[y, z], abs_tol=1e-15)
        assert math.isclose(a([x, x, y, y, z]), u[y] ** 2 * u[z] * P[x, x] + u[x] ** 2 * u[z] * P[y, y]
                            + 4 * u[x] * u[y] * u[z] * P[x, y] + 2 * u[x] * u[y] ** 2 * P[x, z]
                            + 2 * u[x] ** 2 * u[y] * P[y, z], abs_tol=1e-15)
        expect6 = (u[y] ** 2 * u[z] ** 2 * P[x, x] + u[x] ** 2 * u[z] ** 2 * P[y, y] + u[x] ** 2 * u[y] ** 2 * P[z, z]
                   + 4 * u[x] * u[y] * u[z] ** 2 * P[x, y] + 4 * u[x] * u[y] ** 2 * u[z] * P[x, z]
                   + 4 * u[x] ** 2 * u[y] * u[z] * P[y, z])
        assert math.isclose(a([x, x, y, y, z, z]), expect6, abs_tol=1e-15)
        for idx in ([x, x, y], [x, x, y, y], [x, y, y, z, z], [x, x, y, y, z, z]):
            for perm in set(__import__("itertools").permutations(idx)):
                assert math.isclose(a(list(perm)), aneq_pairsum(list(perm), u, P), abs_tol=1e-15)
