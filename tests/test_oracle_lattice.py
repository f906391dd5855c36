"""Pins of the oracle's lattice tables (R1: standard Qian lattices, c_s^2 = 1/3,
P:L63-75) and Hermite bases (R10) against the mathematics that fixes them."""
import itertools
import math

import numpy as np
import pytest

from herm import CS2, he

LATS = ["D2Q9", "D3Q19", "D3Q27"]


@pytest.mark.parametrize("lat", LATS)
def test_isotropy(oracle_mod, lat):
    c, w, opp, _ = oracle_mod.lattice_tables(lat)
    D = 2 if lat == "D2Q9" else 3
    Q = {"D2Q9": 9, "D3Q19": 19, "D3Q27": 27}[lat]
    assert len(w) == Q
    assert np.isclose(w.sum(), 1.0, atol=1e-15)
    assert np.allclose(c.T @ w, 0, atol=1e-16)
    d = np.eye(3)[:D, :D]
    cc = np.einsum("i,ia,ib->ab", w, c, c)[:D, :D]
    assert np.allclose(cc, CS2 * d, atol=1e-15)
    c3 = np.einsum("i,ia,ib,ic->abc", w, c, c, c)
    assert np.allclose(c3, 0, atol=1e-16)
    c4 = np.einsum("i,ia,ib,ic,id->abcd", w, c, c, c, c)[:D, :D, :D, :D]
    iso = CS2 ** 2 * (np.einsum("ab,cd->abcd", d, d) + np.einsum("ac,bd->abcd", d, d)
                      + np.einsum("ad,bc->abcd", d, d))
    assert np.allclose(c4, iso, atol=1e-15)


@pytest.mark.parametrize("lat", LATS)
def test_velocity_set_structure(oracle_mod, lat):
    c, w, opp, _ = oracle_mod.lattice_tables(lat)
    assert len({tuple(v) for v in c}) == len(c)
    assert np.all(np.abs(c) <= 1)
    assert tuple(c[0]) == (0, 0, 0)
    assert np.array_equal(c[opp], -c)
    assert np.array_equal(w[opp], w)
    assert np.array_equal(opp[opp], np.arange(len(c)))
    if lat == "D2Q9":
        assert np.all(c[:, 2] == 0)
        assert {tuple(v[:2]) for v in c} == set(itertools.product([-1, 0, 1], repeat=2))
    if lat == "D3Q27":
        assert {tuple(v) for v in c} == set(itertools.product([-1, 0, 1], repeat=3))
    if lat == "D3Q19":
        assert {tuple(v) for v in c} == {v for v in itertools.product([-1, 0, 1], repeat=3)
                                         if sum(map(abs, v)) <= 2}


@pytest.mark.parametrize("lat", ["D2Q9", "D3Q27"])
def test_weights_are_d1q3_products(oracle_mod, lat):
    c, w, _, _ = oracle_mod.lattice_tables(lat)
    g = {0: 2.0 / 3.0, 1: 1.0 / 6.0}
    D = 2 if lat == "D2Q9" else 3
    for ci, wi in zip(c, w):
        assert math.isclose(wi, np.prod([g[abs(int(ci[a]))] for a in range(D)]), rel_tol=1e-15)


@pytest.mark.parametrize("lat", LATS)
def test_hermite_basis_and_gram(oracle_mod, lat):
    c, w, _, h = oracle_mod.lattice_tables(lat)
    hs = {tuple(v) for v in h}
    assert len(hs) == len(c)
    if lat == "D2Q9":
        assert hs == {(a, b, 0) for a in range(3) for b in range(3)}
    elif lat == "D3Q27":
        assert hs == set(itertools.product(range(3), repeat=3))
    else:
        low = {v for v in itertools.product(range(3), repeat=3) if sum(v) <= 2}
        third = set(itertools.permutations((2, 1, 0)))
        fourth = set(itertools.permutations((2, 2, 0)))
        assert hs == low | third | fourth
    G = np.array([[np.sum(w * he(a, c) * he(b, c)) for b in h] for a in h])
    norms = np.array([math.factorial(v[0]) * math.factorial(v[1]) * math.factorial(v[2]) * CS2 ** sum(v)
                      for v in h])
    if lat in ("D2Q9", "D3Q27"):
        # tensor bases are orthogonal on the lattice with the continuum norms
        assert np.allclose(G, np.diag(norms), atol=1e-15)
    else:
        # D3Q19: orthogonal up to order 2; literal eq-14 basis has the cross
        # term <H_zz, H_xxyy> = -1/27 (R11)
        low = [i for i, v in enumerate(h) if sum(v) <= 2]
        assert np.allclose(G[np.ix_(low, low)], np.diag(norms[low]), atol=1e-15)
        i_zz = [i for i, v in enumerate(h) if tuple(v) == (0, 0, 2)][0]
        i_xxyy = [i for i, v in enumerate(h) if tuple(v) == (2, 2, 0)][0]
        assert math.isclose(G[i_zz, i_xxyy], -1.0 / 27.0, rel_tol=1e-12)
