"""Exact rational brute force of the distribution-form regularized LBM
(SURVEY 8(c) pin 1) -- an independent check of the oracle, test-only.

Everything is a ``fractions.Fraction``: there is no rounding anywhere, so on
tiny grids the result is THE value of the method as the paper defines it, and
the fp64 oracle must agree with it to a few units of rounding.  The code is
written from the paper and the readings of DESIGN.md, not from the oracle, and
it shares nothing with it (or with the CUDA path):

  * velocity sets built by enumeration ({-1,0,1}^D, D3Q19 = |c|^2 <= 2),
    weights as D1Q3 products (D2Q9, D3Q27) or by |c|^2 (D3Q19)  -- R1
  * f^eq by eq 4 written out with c_s^2 = 1/3 (3 c.u + 9/2 (c.u)^2 - 3/2 u^2)
  * Pi^neq = sum_i H2_i f^neq_i (eq 8)
  * projective: eq 9 (f* = f^eq + (1 - 1/tau) w 9/2 H2 : Pi^neq)
  * recursive: eq 14 with the coefficients 1/(a! b! c! c_s^{2n}) (R9) of the
    retained components (R10) and a^neq from the PAIR-SUM closed form
    sum_{p<q} P_{a_p a_q} prod_{r != p,q} u_{a_r} -- the oracle
    uses the Malaspinas recursion, so a wrong recursion index or a
    wrong coefficient shows up here
  * push streaming (eq 7) with periodic wrap, link-wise halfway bounce-back
    with the Ladd lid term 2 w rho (c.u_w)/c_s^2, rho = the node's
    pre-collision density (R12, R13); populations leaving through an open
    face are dropped
  * regularized open faces after the walls (R14): rho from K0 + 2 K- (velocity
    face) or u.n = 1 - (K0 + 2 K-)/rho (pressure face, u_t = 0), f^neq
    bounce-back onto the unknown U+ set, state f^eq + w 9/2 H2 : Pi^neq.
"""
from __future__ import annotations

import itertools
from fractions import Fraction as Fr
from math import factorial

CS2 = Fr(1, 3)
FACES = ("x-", "x+", "y-", "y+", "z-", "z+")


class Lat:
    def __init__(self, name):
        self.name = name
        self.D = 2 if name == "D2Q9" else 3
        cube = list(itertools.product((-1, 0, 1), repeat=self.D))
        if name == "D3Q19":
            cube = [c for c in cube if sum(x * x for x in c) <= 2]
        self.c = [tuple(c) + (0,) * (3 - self.D) for c in cube]
        self.Q = len(self.c)
        w1 = {0: Fr(2, 3), 1: Fr(1, 6), -1: Fr(1, 6)}
        if name == "D3Q19":
            wn = {0: Fr(1, 3), 1: Fr(1, 18), 2: Fr(1, 36)}
            self.w = [wn[sum(x * x for x in c)] for c in self.c]
        else:
            self.w = []
            for c in self.c:
                p = Fr(1)
                for a in range(self.D):
                    p *= w1[c[a]]
                self.w.append(p)
        assert sum(self.w) == 1
        self.opp = [self.c.index(tuple(-x for x in c)) for c in self.c]

    def basis(self, recursive):
        D = self.D
        full = [h + (0,) * (3 - D) for h in itertools.product((0, 1, 2), repeat=D)]
        low = [h for h in full if sum(h) <= 2]
        if not recursive:
            return low
        if self.name == "D3Q19":
            extra = [h for h in full if sorted(h) == [0, 1, 2] or sorted(h) == [0, 2, 2]]
            return low + extra
        return full


def he(order, c):
    return Fr(1) if order == 0 else (Fr(c) if order == 1 else Fr(c * c) - CS2)


def H2(c, a, b):
    return Fr(c[a] * c[b]) - (CS2 if a == b else 0)


def feq(L, rho, u):
    out = []
    uu = sum(x * x for x in u)
    for i, c in enumerate(L.c):
        cu = sum(c[a] * u[a] for a in range(3))
        out.append(L.w[i] * rho * (1 + 3 * cu + Fr(9, 2) * cu * cu - Fr(3, 2) * uu))
    return out


def moments(L, f):
    rho = sum(f)
    j = [sum(L.c[i][a] * f[i] for i in range(L.Q)) for a in range(3)]
    u = [x / rho for x in j]
    Pi = [[sum(H2(L.c[i], a, b) * f[i] for i in range(L.Q)) for b in range(3)] for a in range(3)]
    return rho, u, Pi


def aneq_pairs(h, u, P):
    """sum over index pairs p < q of the multiset h of P_{a_p a_q} prod_{r != p, q} u_{a_r}"""
    idx = [a for a in range(3) for _ in range(h[a])]
    s = Fr(0)
    for p, q in itertools.combinations(range(len(idx)), 2):
        t = P[idx[p]][idx[q]]
        for r in range(len(idx)):
            if r != p and r != q:
                t *= u[idx[r]]
        s += t
    return s


def collide(L, f, tau, recursive):
    rho, u, _ = moments(L, f)
    fe = feq(L, rho, u)
    fneq = [f[i] - fe[i] for i in range(L.Q)]
    P = [[sum(H2(L.c[i], a, b) * fneq[i] for i in range(L.Q)) for b in range(3)] for a in range(3)]
    om = 1 - 1 / tau
    if not recursive:
        return [fe[i] + om * L.w[i] * Fr(9, 2) * sum(H2(L.c[i], a, b) * P[a][b] for a in range(3) for b in range(3))
                for i in range(L.Q)]
    A = {}
    for h in L.basis(True):
        n = sum(h)
        aeq = rho
        for a in range(3):
            aeq *= u[a] ** h[a]
        A[h] = aeq if n < 2 else aeq + om * aneq_pairs(h, u, P)
    out = []
    for i, c in enumerate(L.c):
        s = Fr(0)
        for h, v in A.items():
            n = sum(h)
            s += he(h[0], c[0]) * he(h[1], c[1]) * he(h[2], c[2]) * v / (
                factorial(h[0]) * factorial(h[1]) * factorial(h[2]) * CS2 ** n)
        out.append(L.w[i] * s)
    return out


class Exact:
    """boundary: {face: {"kind": ..., "u": [..], "rho": r}} (Fractions), missing = periodic"""

    def __init__(self, lattice, n, tau, recursive, boundary):
        self.L = Lat(lattice)
        self.n = tuple(n) + (1,) * (3 - len(n))
        self.tau = Fr(tau)
        self.rec = recursive
        self.b = {F: dict(boundary.get(F, {"kind": "periodic"})) for F in FACES}
        if self.L.D == 2:
            self.b["z-"] = self.b["z+"] = {"kind": "periodic"}
        self.nodes = list(itertools.product(range(self.n[0]), range(self.n[1]), range(self.n[2])))
        self.f = {}

    def set_moments(self, mom):
        """mom[node] = (rho, u[3], Pi[3][3]) -> f = w (rho + c.(rho u)/c_s^2 + H2 : Pi / (2 c_s^4))"""
        L = self.L
        for x in self.nodes:
            rho, u, Pi = mom[x]
            self.f[x] = [L.w[i] * (rho + 3 * sum(c[a] * rho * u[a] for a in range(3))
                                   + Fr(9, 2) * sum(H2(c, a, b) * Pi[a][b] for a in range(3) for b in range(3)))
                         for i, c in enumerate(L.c)]

    def get_moments(self):
        return {x: moments(self.L, self.f[x]) for x in self.nodes}

    def step(self):
        L = self.L
        post = {x: collide(L, self.f[x], self.tau, self.rec) for x in self.nodes}
        rho0 = {x: sum(self.f[x]) for x in self.nodes}
        new = {x: [None] * L.Q for x in self.nodes}
        for x in self.nodes:
            for i, c in enumerate(L.c):
                d = list(x)
                wall = opened = False
                lid = Fr(0)
                for a in range(3):
                    d[a] = x[a] + c[a]
                    F = None
                    if d[a] < 0:
                        F = FACES[2 * a]
                    elif d[a] >= self.n[a]:
                        F = FACES[2 * a + 1]
                    if F is None:
                        continue
                    k = self.b[F]["kind"]
                    if k == "periodic":
                        d[a] %= self.n[a]
                    elif k in ("wall", "moving_wall"):
                        wall = True
                        if k == "moving_wall":
                            uw = [Fr(v) for v in self.b[F]["u"]]
                            lid += 2 * L.w[i] * rho0[x] * sum(c[q] * uw[q] for q in range(3)) / CS2
                    else:
                        opened = True
                if wall:
                    new[x][L.opp[i]] = post[x][i] - lid
                elif not opened:
                    new[tuple(d)][i] = post[x][i]
        for F in FACES:
            spec = self.b[F]
            if spec["kind"] not in ("velocity", "pressure"):
                continue
            ax = FACES.index(F) // 2
            fixed = 0 if FACES.index(F) % 2 == 0 else self.n[ax] - 1
            nrm = [0, 0, 0]
            nrm[ax] = 1 if FACES.index(F) % 2 == 0 else -1
            for x in self.nodes:
                if x[ax] == fixed:
                    new[x] = self._open(new[x], spec, nrm)
        for x in self.nodes:
            assert all(v is not None for v in new[x]), (x, new[x])  # every population arrived or was rebuilt
        self.f = new

    def _open(self, f, spec, nrm):
        L = self.L
        cn = [sum(c[a] * nrm[a] for a in range(3)) for c in L.c]
        S = sum(f[i] for i in range(L.Q) if cn[i] == 0) + 2 * sum(f[i] for i in range(L.Q) if cn[i] < 0)
        if spec["kind"] == "velocity":
            u = [Fr(v) for v in spec["u"]]
            rho = S / (1 - sum(u[a] * nrm[a] for a in range(3)))
        else:
            rho = Fr(spec["rho"])
            un = 1 - S / rho
            u = [un * nrm[a] for a in range(3)]
        fe = feq(L, rho, u)
        fneq = [None if cn[i] > 0 else f[i] - fe[i] for i in range(L.Q)]
        for i in range(L.Q):
            if cn[i] > 0:
                fneq[i] = fneq[L.opp[i]]
        P = [[sum(H2(L.c[i], a, b) * fneq[i] for i in range(L.Q)) for b in range(3)] for a in range(3)]
        return [fe[i] + L.w[i] * Fr(9, 2) * sum(H2(L.c[i], a, b) * P[a][b] for a in range(3) for b in range(3))
                for i in range(L.Q)]


def abi_moments(ex):
    """[M][nz][ny][nx] (3D) / [M][ny][nx] (2D) lists of Fractions in the ABI order"""
    D = ex.L.D
    mom = ex.get_moments()
    nx, ny, nz = ex.n
    slots = [("r",), ("u", 0), ("u", 1)] + ([("u", 2)] if D == 3 else [])
    if D == 2:
        slots += [("P", 0, 0), ("P", 1, 1), ("P", 0, 1)]
    else:
        slots += [("P", 0, 0), ("P", 1, 1), ("P", 2, 2), ("P", 0, 1), ("P", 0, 2), ("P", 1, 2)]
    out = []
    for s in slots:
        plane = []
        for z in range(nz):
            rows = []
            for y in range(ny):
                row = []
                for x in range(nx):
                    rho, u, Pi = mom[(x, y, z)]
                    row.append(rho if s[0] == "r" else (u[s[1]] if s[0] == "u" else Pi[s[1]][s[2]]))
                rows.append(row)
            plane.append(rows)
        out.append(plane if D == 3 else plane[0])
    return out
