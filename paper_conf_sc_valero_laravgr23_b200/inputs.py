"""Seeded synthetic inputs shared by the CUDA path's tests/bench and the oracle.

This module holds NO arithmetic of the method (no equilibrium, collision,
reconstruction or streaming): only initial moment fields (rho, u, Pi) and
boundary specifications with the shapes of the paper's workloads (channel
flow) and of BASELINE.json's configs (Poiseuille channel, lid-driven
cavity, Taylor-Green vortex).  Fields are returned in the ABI moment layout
  2D: [6][ny][nx]   rho ux uy Pxx Pyy Pxy
  3D: [10][nz][ny][nx]  rho ux uy uz Pxx Pyy Pzz Pxy Pxz Pyz
where Pi is the Hermite second moment (eq 3) and u the velocity.

The recipe: perturbations use
numpy.random.default_rng(seed) (default 20231112), a sum of 4 random-phase
Fourier modes, amplitude 1e-3 on rho and 1e-3*U on u, plus a 1e-4*U^2
random symmetric non-equilibrium part in Pi so that every Hermite term is
exercised.
"""
from __future__ import annotations

import math

import numpy as np

SEED = 20231112
CS2 = 1.0 / 3.0


def n_moments(D: int) -> int:
    return 6 if D == 2 else 10


class _Modes:
    """Sum of nmodes random-phase low-wavenumber Fourier modes on a periodic
    grid (slowest axis first).  The random parameters are drawn at
    construction (phase, then one wavenumber 1..3 per axis, per mode); the
    field is evaluated on any range [lo, hi) of the slowest axis, so a slab
    of a multi-GPU decomposition gets exactly its part of the global field
    without building the rest."""

    def __init__(self, rng, grid, amp, nmodes=4):
        self.grid, self.amp, self.nmodes = tuple(grid), amp, nmodes
        self.params = []
        for _ in range(nmodes):
            ph = rng.uniform(0, 2 * np.pi)
            ks = [int(rng.integers(1, 4)) for _ in grid]
            self.params.append((ph, ks))

    def eval(self, lo=0, hi=None):
        hi = self.grid[0] if hi is None else hi
        shape = (hi - lo,) + self.grid[1:]
        # cos(ph + sum_a 2 pi k_a x_a / n_a) = Re(P(x_0..x_{D-2}) F(x_{D-1})) with
        # per-axis phase factors: the mode sum is one small real matrix product
        # [Re P | -Im P] @ [Re F ; Im F] (no full-size argument or cos array)
        L = np.empty((int(np.prod(shape[:-1])), 2 * self.nmodes))
        R = np.empty((2 * self.nmodes, shape[-1]))
        for m, (ph, ks) in enumerate(self.params):
            P = np.exp(1j * ph) * np.ones(shape[:-1], dtype=complex)
            for a, (k, n) in enumerate(zip(ks[:-1], self.grid[:-1])):
                idx = np.arange(lo, hi) if a == 0 else np.arange(n)
                f = np.exp(2j * np.pi * k * idx / n)
                P = P * f.reshape([-1 if b == a else 1 for b in range(len(shape) - 1)])
            F = np.exp(2j * np.pi * ks[-1] * np.arange(shape[-1]) / self.grid[-1])
            L[:, 2 * m], L[:, 2 * m + 1] = P.real.reshape(-1), -P.imag.reshape(-1)
            R[2 * m], R[2 * m + 1] = F.real, F.imag
        return (self.amp / self.nmodes) * (L @ R).reshape(shape)


def _modes(rng, grid, amp, nmodes=4):
    """Sum of nmodes random-phase low-wavenumber Fourier modes on a periodic grid."""
    return _Modes(rng, grid, amp, nmodes).eval()


def pack(rho, u, Pi) -> np.ndarray:
    """rho [grid], u [D][grid], Pi [D][D][grid] -> ABI moment array."""
    D = len(u)
    if D == 2:
        return np.stack([rho, u[0], u[1], Pi[0][0], Pi[1][1], Pi[0][1]]).astype(np.float64)
    return np.stack([rho, u[0], u[1], u[2], Pi[0][0], Pi[1][1], Pi[2][2],
                     Pi[0][1], Pi[0][2], Pi[1][2]]).astype(np.float64)


def _grid(D, nx, ny, nz):
    return (ny, nx) if D == 2 else (nz, ny, nx)


def perturbed_rest(D, nx, ny, nz=1, U=0.05, seed=SEED, pi_neq=True, lo=0, hi=None, chunk=16):
    """Rest state (rho=1, u=0) plus seeded random-phase perturbations.
    lo, hi: range of the slowest axis (z in 3D, y in 2D) to return -- a slab
    of the global field, generated in chunks of `chunk` planes straight into
    the output (bench: one 1024 x 1024 x 128 slab per GPU)."""
    rng = np.random.default_rng(seed)
    g = _grid(D, nx, ny, nz)
    hi = g[0] if hi is None else hi
    m_rho = _Modes(rng, g, 1e-3)
    m_u = [_Modes(rng, g, 1e-3 * U) for _ in range(D)]
    m_pi = {}
    for a in range(D):
        for b in range(a, D):
            m_pi[(a, b)] = _Modes(rng, g, 1e-4 * U * U) if pi_neq else None
    out = np.empty((n_moments(D), hi - lo) + g[1:])
    for c0 in range(lo, hi, chunk):
        c1 = min(hi, c0 + chunk)
        o = out[:, c0 - lo:c1 - lo]
        rho = o[0]
        rho[...] = m_rho.eval(c0, c1)
        rho += 1.0
        u = []
        for a in range(D):
            o[1 + a] = m_u[a].eval(c0, c1)
            u.append(o[1 + a])
        for (a, b), slot in _pi_slots(D).items():
            v = o[slot]
            if pi_neq:
                v[...] = m_pi[(a, b)].eval(c0, c1)
                v += rho * u[a] * u[b]
            else:
                v[...] = rho * u[a] * u[b]
    return out


def _pi_slots(D):
    """ABI slot of Pi_ab (a <= b), in the generation order of perturbed_rest"""
    if D == 2:
        return {(0, 0): 3, (0, 1): 5, (1, 1): 4}
    return {(0, 0): 4, (0, 1): 7, (0, 2): 8, (1, 1): 5, (1, 2): 9, (2, 2): 6}


def smooth_state(D, nx, ny, nz=1, U=0.05, seed=SEED, mean_u=None):
    """Smooth seeded flow of order U: 4 random-phase modes on every moment
    (rho: 1e-2, u: U, Pi^neq: 1e-3 U) -- parity tests (every Hermite term
    and every velocity component is O(U), so the per-group metric is not
    dominated by absolute rounding of near-zero fields).  mean_u: a uniform
    velocity added to u (periodic runs long enough for the modes to decay
    viscously keep an O(U) field)."""
    rng = np.random.default_rng(seed)
    g = _grid(D, nx, ny, nz)
    rho = 1.0 + _modes(rng, g, 1e-2)
    u = [_modes(rng, g, U) for _ in range(D)]
    if mean_u is not None:
        u = [u[a] + mean_u[a] for a in range(D)]
    Pi = [[None] * D for _ in range(D)]
    for a in range(D):
        for b in range(a, D):
            Pi[a][b] = Pi[b][a] = rho * u[a] * u[b] + _modes(rng, g, 1e-3 * U)
    return pack(rho, u, Pi)


def random_state(D, nx, ny, nz=1, U=0.05, seed=SEED):
    """Non-smooth seeded state: i.i.d. noise on every moment (parity stress test)."""
    rng = np.random.default_rng(seed)
    g = _grid(D, nx, ny, nz)
    rho = 1.0 + 1e-2 * rng.standard_normal(g)
    u = [U * rng.uniform(-1, 1, g) for _ in range(D)]
    Pi = [[None] * D for _ in range(D)]
    for a in range(D):
        for b in range(a, D):
            Pi[a][b] = Pi[b][a] = rho * u[a] * u[b] + 1e-3 * U * rng.standard_normal(g)
    return pack(rho, u, Pi)


def poiseuille_profile(ny, U):
    """u_x(y) = 4U (y+1/2)(H-y-1/2)/H^2, walls halfway (y=-1/2, H-1/2), H=ny."""
    y = np.arange(ny) + 0.5
    return 4.0 * U * y * (ny - y) / ny ** 2


def poiseuille_state(nx, ny, U, tau, rho_out=1.0):
    """Analytic 2D Poiseuille state (pin 7): parabolic u_x, linear pressure,
    Pi = rho u u + Pi^neq with Pi^neq_xy = -rho c_s^2 tau du_x/dy."""
    nu = CS2 * (tau - 0.5)
    H = float(ny)
    dpdx = -8.0 * nu * U * rho_out / H ** 2
    x = np.arange(nx)[None, :].repeat(ny, 0).astype(float)
    yc = (np.arange(ny) + 0.5)[:, None].repeat(nx, 1)
    ux = 4.0 * U * yc * (H - yc) / H ** 2
    duy = 4.0 * U * (H - 2 * yc) / H ** 2
    rho = rho_out + dpdx * (x - (nx - 1)) / CS2
    uy = np.zeros_like(ux)
    Pxy = rho * ux * uy - rho * CS2 * tau * duy
    Pi = [[rho * ux * ux, Pxy], [Pxy, rho * uy * uy]]
    return pack(rho, [ux, uy], Pi)


def taylor_green_2d(n, U, tau, t=0.0):
    """u = U(-cos kx sin ky, sin kx cos ky) e^{-2 nu k^2 t}, periodic n x n."""
    nu = CS2 * (tau - 0.5)
    k = 2 * np.pi / n
    y, x = np.meshgrid(np.arange(n), np.arange(n), indexing="ij")
    d = math.exp(-2 * nu * k * k * t)
    ux = -U * np.cos(k * x) * np.sin(k * y) * d
    uy = U * np.sin(k * x) * np.cos(k * y) * d
    p = -0.25 * U * U * d * d * (np.cos(2 * k * x) + np.cos(2 * k * y))
    rho = 1.0 + p / CS2
    Pi = [[rho * ux * ux, rho * ux * uy], [rho * ux * uy, rho * uy * uy]]
    return pack(rho, [ux, uy], Pi)


def taylor_green_3d(n, U, tau=0.6):
    """C3 initial state: u = U(sin x cos y cos z, -cos x sin y cos z, 0),
    p = rho0 U^2/16 (cos2x + cos2y)(cos2z + 2), rho = 1 + p/c_s^2, Pi = rho u u."""
    z, y, x = np.meshgrid(*[2 * np.pi * np.arange(n) / n] * 3, indexing="ij")
    ux = U * np.sin(x) * np.cos(y) * np.cos(z)
    uy = -U * np.cos(x) * np.sin(y) * np.cos(z)
    uz = np.zeros_like(ux)
    p = U * U / 16.0 * (np.cos(2 * x) + np.cos(2 * y)) * (np.cos(2 * z) + 2.0)
    rho = 1.0 + p / CS2
    u = [ux, uy, uz]
    Pi = [[rho * u[a] * u[b] for b in range(3)] for a in range(3)]
    return pack(rho, u, Pi)


def taylor_green_3d_extruded(n, m, U, tau, axis=2):
    """2D Taylor-Green field in the plane normal to `axis` (n x n, periodic),
    extruded uniformly over m nodes along `axis` (an exact Navier-Stokes
    solution in 3D).  Returns the 3D ABI array [10][nz][ny][nx]."""
    k = 2 * np.pi / n
    p, q = [a for a in range(3) if a != axis]
    ext = [n, n, n]
    ext[axis] = m
    nx, ny, nz = ext
    z, y, x = np.meshgrid(np.arange(nz), np.arange(ny), np.arange(nx), indexing="ij")
    X = [x, y, z]
    up = -U * np.cos(k * X[p]) * np.sin(k * X[q])
    uq = U * np.sin(k * X[p]) * np.cos(k * X[q])
    pr = -0.25 * U * U * (np.cos(2 * k * X[p]) + np.cos(2 * k * X[q]))
    rho = 1.0 + pr / CS2
    u = [np.zeros_like(rho) for _ in range(3)]
    u[p], u[q] = up, uq
    Pi = [[rho * u[a] * u[b] for b in range(3)] for a in range(3)]
    return pack(rho, u, Pi)


def channel3d_profile(ny, nz, U):
    """C5 inlet: u_x = 16 U yh(1-yh) zh(1-zh), yh = (y+1/2)/ny; face array [nz][ny][3]."""
    yh = (np.arange(ny) + 0.5) / ny
    zh = (np.arange(nz) + 0.5) / nz
    ux = 16.0 * U * (zh[:, None] * (1 - zh[:, None])) * (yh[None, :] * (1 - yh[None, :]))
    out = np.zeros((nz, ny, 3))
    out[..., 0] = ux
    return out
