"""An independent, tiny MOMENT-FORM stepper in numpy (tests only).

Used to pin the oracle (distribution form, push streaming, recursion loop)
against the paper's own moment representation: state = moments,
collision eqs 10 / 12-13 with the pair-sum closed forms, reconstruction eqs
11 / 14, PULL streaming with numpy.roll, moments eqs 1-3.  Periodic, wall and
moving-wall faces only (open faces are pinned by the Poiseuille tests).
Shares no code with ``oracle/`` or with the CUDA path.
"""
import itertools

import numpy as np

from herm import CS2, he, idx_of, aneq_pairsum

import math

FACES = ("x-", "x+", "y-", "y+", "z-", "z+")


def step(m, lat_tables, reg, tau, boundary, D):
    """One timestep of the moment representation.  m: ABI moments [M][grid]."""
    c, w, opp, herm = lat_tables
    grid = m.shape[1:]
    rho = m[0]
    u = [m[1 + a] for a in range(D)] + [np.zeros(grid)] * (3 - D)
    Pi = [[np.zeros(grid)] * 3 for _ in range(3)]
    if D == 2:
        Pi[0][0], Pi[1][1], Pi[0][1] = m[3], m[4], m[5]
        Pi[1][0] = m[5]
    else:
        Pi[0][0], Pi[1][1], Pi[2][2] = m[4], m[5], m[6]
        Pi[0][1] = Pi[1][0] = m[7]
        Pi[0][2] = Pi[2][0] = m[8]
        Pi[1][2] = Pi[2][1] = m[9]
    om = 1 - 1 / tau
    P = [[Pi[a][b] - rho * u[a] * u[b] for b in range(3)] for a in range(3)]  # Pi^neq
    # collided Hermite coefficients
    if reg == "projective":
        keep = [h for h in herm if sum(h) <= 2]
    else:
        keep = list(herm)
    fstar = []
    for i in range(len(w)):
        s = np.zeros(grid)
        for h in keep:
            h = tuple(int(v) for v in h)
            idx = idx_of(h)
            n = len(idx)
            aeq = rho.copy()
            for a in idx:
                aeq = aeq * u[a]
            if n <= 1:
                A = aeq
            elif n == 2:
                A = aeq + om * P[idx[0]][idx[1]]
            else:
                ane = np.zeros(grid)
                for p, q in itertools.combinations(range(n), 2):
                    t = P[idx[p]][idx[q]]
                    for k in range(n):
                        if k != p and k != q:
                            t = t * u[idx[k]]
                    ane = ane + t
                A = aeq + om * ane
            coef = 1.0 / (math.factorial(h[0]) * math.factorial(h[1]) * math.factorial(h[2]) * CS2 ** n)
            s = s + float(he(h, c[i])) * coef * A
        fstar.append(w[i] * s)
    # pull streaming
    ext = grid[::-1]  # (nx, ny[, nz])
    coords = np.meshgrid(*[np.arange(n) for n in grid], indexing="ij")[::-1]  # x, y[, z]
    fnew = []
    for i in range(len(w)):
        ci = c[i][:D]
        shifted = np.roll(fstar[i], shift=tuple(int(v) for v in ci[::-1]), axis=tuple(range(D)))
        out_wall = np.zeros(grid, dtype=bool)
        lid = np.zeros(grid)
        for a in range(D):
            if ci[a] == 0:
                continue
            F = 2 * a if ci[a] > 0 else 2 * a + 1  # source beyond the lower / upper face
            edge = (coords[a] == 0) if ci[a] > 0 else (coords[a] == ext[a] - 1)
            spec = boundary.get(FACES[F], {"kind": "periodic"})
            if spec["kind"] in ("wall", "moving_wall"):
                out_wall |= edge
                if spec["kind"] == "moving_wall":
                    uw = np.zeros(3)
                    uw[:len(spec["u"])] = spec["u"]
                    # f_i(x) = f*_opp(i)(x) + 2 w_i rho (c_i . u_w) / c_s^2  (Ladd)
                    lid = lid + np.where(edge, 2 * w[i] * rho * float(c[i] @ uw) / CS2, 0.0)
        fnew.append(np.where(out_wall, fstar[opp[i]] + lid, shifted))
    fnew = np.array(fnew)
    # moments eqs 1-3
    r = fnew.sum(0)
    j = np.einsum("ia,i...->a...", c.astype(float), fnew)
    uu = j / r
    PP = np.einsum("ia,ib,i...->ab...", c.astype(float), c.astype(float), fnew) - CS2 * r * np.eye(3)[:, :, None].reshape((3, 3) + (1,) * len(grid))
    if D == 2:
        return np.stack([r, uu[0], uu[1], PP[0, 0], PP[1, 1], PP[0, 1]])
    return np.stack([r, uu[0], uu[1], uu[2], PP[0, 0], PP[1, 1], PP[2, 2], PP[0, 1], PP[0, 2], PP[1, 2]])
