"""SURVEY 8(c) pin 1: the fp64 oracle against an EXACT rational brute force
(tests/exact_lbm.py, Python fractions, written independently from the paper)
on tiny grids, every lattice x regularization, every boundary kind:
periodic wrap, halfway bounce-back walls, moving walls (Ladd), regularized
velocity inlet and pressure outlet -- including the EDGE nodes where an open
face meets a wall or a moving wall, which no analytic solution pins
(DESIGN.md "parity unpinned" before this test).

Inputs are dyadic rationals (exactly representable in fp64), so the only
difference between the two is the oracle's rounding.  The moments are sums of
O(1) populations, so the rounding floor is absolute, a few ulp(1) = 2.2e-16
(a Q-term sum of O(1) values after 2-3 steps): measured <= 6 ulp(1) = 1.3e-15
on every case; the bound is 8 ulp(1) = 1.8e-15 on every moment.  Any
dropped term, wrong sign, index or coefficient changes some moment by
O(U^3) ~ 1e-5 or more.
"""
import itertools
import random
from fractions import Fraction as Fr

import numpy as np
import pytest

import exact_lbm as E

TOL_ABS = 8 * np.finfo(np.float64).eps


def rand_moments(D, n, seed):
    rng = random.Random(seed)
    mom = {}
    for x in itertools.product(range(n[0]), range(n[1]), range(n[2] if D == 3 else 1)):
        rho = 1 + Fr(rng.randint(-40, 40), 2048)
        u = [Fr(rng.randint(-100, 100), 2048) for _ in range(D)] + [Fr(0)] * (3 - D)
        Pi = [[rho * u[a] * u[b] for b in range(3)] for a in range(3)]
        for a in range(D):
            for b in range(a, D):
                d = Fr(rng.randint(-50, 50), 1 << 16)
                Pi[a][b] += d
                if a != b:
                    Pi[b][a] += d
        mom[x] = (rho, u, Pi)
    return mom


def cases():
    out = []
    for lat in ("D2Q9", "D3Q19", "D3Q27"):
        D = 2 if lat == "D2Q9" else 3
        z0 = Fr(0)
        # (a) channel: velocity inlet x-, pressure outlet x+, wall y-, moving wall y+ (and z walls / lid)
        chan = {"x-": {"kind": "velocity", "u": [Fr(3, 128), Fr(1, 256), z0 if D == 2 else Fr(-1, 512)]},
                "x+": {"kind": "pressure", "rho": Fr(1013, 1024)},
                "y-": {"kind": "wall"},
                "y+": {"kind": "moving_wall", "u": [Fr(1, 16), z0, z0 if D == 2 else Fr(1, 64)]}}
        if D == 3:
            chan["z-"] = {"kind": "wall"}
            chan["z+"] = {"kind": "moving_wall", "u": [z0, Fr(1, 32), z0]}
        out.append((lat, "channel_x", (4, 3, 1) if D == 2 else (4, 3, 3), chan))
        if D == 2:
            # (b) periodic x, cavity walls in y
            out.append((lat, "periodic_x_lid", (3, 4, 1),
                        {"y-": {"kind": "wall"}, "y+": {"kind": "moving_wall", "u": [Fr(-1, 32), z0, z0]}}))
            out.append((lat, "periodic", (3, 3, 1), {}))
        else:
            # (b) open faces on y (pressure inlet side low), walls on x (one moving), periodic z
            out.append((lat, "channel_y", (3, 4, 3),
                        {"y-": {"kind": "velocity", "u": [Fr(1, 512), Fr(5, 128), Fr(-1, 256)]},
                         "y+": {"kind": "pressure", "rho": Fr(1025, 1024)},
                         "x-": {"kind": "wall"}, "x+": {"kind": "moving_wall", "u": [z0, Fr(1, 64), Fr(1, 32)]}}))
            out.append((lat, "periodic", (3, 3, 3), {}))
    return out


def _float_boundary(b):
    def conv(v):
        if isinstance(v, str):
            return v
        if isinstance(v, list):
            return [float(q) for q in v]
        return float(v)
    return {F: {k: conv(v) for k, v in spec.items()} for F, spec in b.items()}


@pytest.mark.parametrize("reg", ["projective", "recursive"])
@pytest.mark.parametrize("lat,name,n,bnd", cases(), ids=lambda v: v if isinstance(v, str) else None)
def test_oracle_matches_exact_rationals(oracle_mod, lat, name, n, bnd, reg):
    D = 2 if lat == "D2Q9" else 3
    # exact D3Q*-R denominators grow ~8x per step (u^6 terms): 2 steps keep the
    # brute force at seconds; every other case runs 3
    steps = 2 if (D == 3 and reg == "recursive") else 3
    tau = Fr(3, 4)
    ex = E.Exact(lat, n, tau, reg == "recursive", bnd)
    ex.set_moments(rand_moments(D, n, seed=sum(map(ord, lat + name))))
    m0 = np.array(E.abi_moments(ex), dtype=np.float64)  # dyadic: exact in fp64
    for _ in range(steps):
        ex.step()
    ref = np.array(E.abi_moments(ex), dtype=np.float64)
    o = oracle_mod.Oracle(lat, n[0], n[1], n[2], float(tau), reg, _float_boundary(bnd))
    o.set_moments(m0)
    o.step(steps)
    got = o.get_moments()
    err = np.abs(got - ref).max()
    assert err <= TOL_ABS, f"{lat}-{reg} {name}: oracle vs exact rationals {err:.3e}"
    # the case really moves: the state after the steps differs from the start
    assert np.abs(ref - m0).max() > 1e-4
