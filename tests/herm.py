"""Independent closed forms used by the oracle pins (tests only).

Nothing here is imported by the oracle or by the CUDA path.  These are the
*other* formulas the paper's method must agree with:
  - the textbook second-order BGK equilibrium 1 + 3cu + 9/2 (cu)^2 - 3/2 u^2
    (eq 4 with c_s^2 = 1/3 written out; Alg. 1 line 24 P:L170 corrected, R2),
  - the D1Q3 product equilibrium (tau = 1 recursive reduction, SURVEY pin 5),
  - the moment-form projective collision eqs 10-11,
  - the NON-recursive pair-sum closed form of Malaspinas' recursion
    (SURVEY App. A), against which the oracle's recursion loop is checked.
"""
import itertools
import math

import numpy as np

CS2 = 1.0 / 3.0


def he1(order, c):
    c = np.asarray(c, dtype=float)
    if order == 0:
        return np.ones_like(c)
    if order == 1:
        return c
    return c * c - CS2


def he(h, c):
    """tensor-product Hermite polynomial for component h=(a,b,c) at velocities c[...,3]"""
    c = np.asarray(c, dtype=float)
    return he1(h[0], c[..., 0]) * he1(h[1], c[..., 1]) * he1(h[2], c[..., 2])


def textbook_feq(c, w, rho, u):
    cu = c @ u
    return w * rho * (1 + 3 * cu + 4.5 * cu * cu - 1.5 * (u @ u))


def d1q3_product(c, rho, u, D=3):
    """rho * prod_{a<D} g(c_a, u_a), g(0,u) = 2/3 - u^2, g(+-1,u) = (1 +- 3u + 3u^2)/6"""
    out = np.full(len(c), rho, dtype=float)
    for a in range(D):
        ca = c[:, a]
        g = np.where(ca == 0, 2.0 / 3.0 - u[a] ** 2, (1 + 3 * ca * u[a] + 3 * u[a] ** 2) / 6.0)
        out *= g
    return out


def moments(c, f):
    """eqs 1-3 over the lattice dimensions (z entries zero for D2Q9)"""
    D = 2 if np.all(c[:, 2] == 0) else 3
    rho = f.sum()
    j = c.T @ f
    u = j / rho
    Pi = np.einsum("i,ia,ib->ab", f, c, c) - CS2 * rho * np.diag([1.0] * D + [0.0] * (3 - D))
    return rho, u, Pi


def aneq_pairsum(idx, u, P):
    """sum over index pairs (i<j) of P[a_i, a_j] * prod_{k not in {i,j}} u[a_k]"""
    n = len(idx)
    s = 0.0
    for i, j in itertools.combinations(range(n), 2):
        p = P[idx[i], idx[j]]
        for k in range(n):
            if k != i and k != j:
                p *= u[idx[k]]
        s += p
    return s


def idx_of(h):
    return [a for a in range(3) for _ in range(h[a])]


def recursive_moment_form(c, w, herm, tau, rho, u, Pneq):
    """eqs 10, 12-14 with the pair-sum closed forms: coefficients A*_h and f*."""
    om = 1 - 1 / tau
    A = {}
    for h in herm:
        h = tuple(int(v) for v in h)
        idx = idx_of(h)
        n = len(idx)
        aeq = rho * np.prod([u[a] for a in idx]) if n else rho
        A[h] = aeq if n <= 1 else aeq + om * aneq_pairsum(idx, u, Pneq)
    f = np.zeros(len(c))
    for h, a in A.items():
        n = sum(h)
        coef = 1.0 / (math.factorial(h[0]) * math.factorial(h[1]) * math.factorial(h[2]) * CS2 ** n)
        f += he(h, c) * coef * a
    return A, w * f


def projective_moment_form(c, w, tau, rho, u, Pneq):
    """eqs 10-11: Pi* = rho uu + (1-1/tau) Pi^neq; f* = w(rho + c.rho u/cs2 + H2:Pi*/(2cs4))"""
    Pstar = rho * np.outer(u, u) + (1 - 1 / tau) * Pneq
    H2 = np.einsum("ia,ib->iab", c, c) - CS2 * np.eye(3)
    return w * (rho + (c @ (rho * u)) / CS2 + np.einsum("iab,ab->i", H2, Pstar) / (2 * CS2 ** 2))
