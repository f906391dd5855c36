"""The BASELINE.json workloads C1..C5, as plain data.

Each config names the lattice, regularization, grid, tau, boundary faces and
an initial-state recipe from ``inputs``.  No arithmetic of the method here.
"""
from __future__ import annotations

from dataclasses import dataclass, field

from . import inputs


@dataclass
class Config:
    name: str
    lattice: str
    regularization: str
    nx: int
    ny: int
    nz: int
    tau: float
    precision: str
    boundary: dict = field(default_factory=dict)
    init: str = "perturbed_rest"
    U: float = 0.05
    steps: int = 1000

    @property
    def D(self):
        return 2 if self.lattice == "D2Q9" else 3

    @property
    def nodes(self):
        return self.nx * self.ny * (1 if self.D == 2 else self.nz)

    def initial_moments(self, seed=inputs.SEED, lo=0, hi=None):
        """ABI moments of the initial state; lo, hi: only layers [lo, hi) of the
        slowest axis (z in 3D, y in 2D) -- one rank's slab"""
        if self.init == "poiseuille":
            return inputs.poiseuille_state(self.nx, self.ny, self.U, self.tau)[:, lo:hi]
        if self.init == "taylor_green_3d":
            return inputs.taylor_green_3d(self.nx, self.U, self.tau)[:, lo:hi]
        return inputs.perturbed_rest(self.D, self.nx, self.ny, self.nz, self.U, seed, lo=lo, hi=hi)


def _walls(D, lid_face=None, U=0.0):
    faces = ["x-", "x+", "y-", "y+"] + (["z-", "z+"] if D == 3 else [])
    b = {f: {"kind": "wall"} for f in faces}
    if lid_face:
        b[lid_face] = {"kind": "moving_wall", "u": [U, 0.0, 0.0]}
    return b


def c1():
    U, ny = 0.05, 64
    return Config("C1", "D2Q9", "projective", 128, ny, 1, 0.8, "fp64",
                  {"x-": {"kind": "velocity", "u_profile": inputs.poiseuille_profile(ny, U)[:, None].repeat(2, 1) * [1, 0]},
                   "x+": {"kind": "pressure", "rho": 1.0},
                   "y-": {"kind": "wall"}, "y+": {"kind": "wall"}},
                  init="poiseuille", U=U, steps=1000)


def c2(precision="fp64", n=4096):
    U = 0.1
    tau = 0.5 + 3 * U * n / 1000.0
    return Config("C2", "D2Q9", "recursive", n, n, 1, tau, precision, _walls(2, "y+", U), U=U)


def c3(n=256):
    return Config("C3", "D3Q19", "projective", n, n, n, 0.6, "fp64", {}, init="taylor_green_3d", U=0.05)


def c4(n=512, precision="fp32"):
    U = 0.1
    tau = 0.5 + 3 * U * n / 1000.0
    return Config("C4", "D3Q27", "recursive", n, n, n, tau, precision, _walls(3, "y+", U), U=U)


def c5(nx=1024, ny=1024, nz=1024, U=0.05):
    b = {"x-": {"kind": "velocity", "u_profile": inputs.channel3d_profile(ny, nz, U)},
         "x+": {"kind": "pressure", "rho": 1.0},
         "y-": {"kind": "wall"}, "y+": {"kind": "wall"},
         "z-": {"kind": "wall"}, "z+": {"kind": "wall"}}
    return Config("C5", "D3Q19", "recursive", nx, ny, nz, 0.6, "fp64", b, U=U)


ALL = {"C1": c1, "C2": c2, "C3": c3, "C4": c4, "C5": c5}
