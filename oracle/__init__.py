"""CPU oracle for the MR-LBM hot path -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its
``cpu_baseline`` leg and ``--impl reference``) may import this package.  The
product package ``paper_conf_sc_valero_laravgr23_b200`` never imports it and
shares no code with it.

The arithmetic lives in ``mrlbm_oracle.c`` (plain C, fp64, distribution form;
every function cites the PAPER.md passage it follows).  This module only
compiles it with gcc and marshals arguments through ctypes.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from pathlib import Path

import numpy as np

_HERE = Path(__file__).resolve().parent
_SRC = _HERE / "mrlbm_oracle.c"
_LIB = _HERE / "liboracle.so"

LATTICES = {"D2Q9": 0, "D3Q19": 1, "D3Q27": 2}
REGS = {"projective": 0, "recursive": 1, "bgk": 2}
BC = {"periodic": 0, "wall": 1, "moving_wall": 2, "velocity": 3, "pressure": 4,
      "velocity_fd": 5, "pressure_fd": 6}
FACES = ("x-", "x+", "y-", "y+", "z-", "z+")


def build(force: bool = False) -> Path:
    """Compile the oracle shared library (gcc -O2 -fopenmp)."""
    if force or not _LIB.exists() or _LIB.stat().st_mtime < _SRC.stat().st_mtime:
        tmp = _LIB.with_suffix(f".{os.getpid()}.tmp")
        subprocess.run(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-std=c99",
                        "-o", str(tmp), str(_SRC), "-lm"], check=True)
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        L = ctypes.CDLL(str(build()))
        P = ctypes.c_void_p
        dp = ctypes.POINTER(ctypes.c_double)
        ip = ctypes.POINTER(ctypes.c_int)
        L.oracle_create.restype = P
        L.oracle_create.argtypes = [ctypes.c_int, ctypes.c_int64, ctypes.c_int64, ctypes.c_int64,
                                    ctypes.c_double, ctypes.c_int, ip, dp, dp,
                                    ctypes.POINTER(dp), ctypes.c_int]
        L.oracle_destroy.argtypes = [P]
        for name in ("oracle_set_moments", "oracle_set_f"):
            getattr(L, name).argtypes = [P, dp]
        for name in ("oracle_get_moments", "oracle_get_f", "oracle_get_populations"):
            getattr(L, name).argtypes = [P, dp]
        L.oracle_step.argtypes = [P, ctypes.c_int64]
        L.oracle_collide_node.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_double, dp, dp]
        L.oracle_feq.argtypes = [ctypes.c_int, ctypes.c_double, dp, dp]
        L.oracle_lattice.argtypes = [ctypes.c_int, ip, dp, ip, ip]
        L.oracle_lattice.restype = ctypes.c_int
        L.oracle_aneq.argtypes = [ip, ctypes.c_int, dp, dp]
        L.oracle_aneq.restype = ctypes.c_double
        L.oracle_max_threads.restype = ctypes.c_int
        _lib = L
    return _lib


def _dp(a: np.ndarray):
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_double))


def max_threads() -> int:
    return lib().oracle_max_threads()


def lattice_tables(lattice: str):
    """(c[Q,3], w[Q], opp[Q], hermite[Q,3]) of the oracle's own tables."""
    c = np.zeros(81, dtype=np.int32)
    h = np.zeros(81, dtype=np.int32)
    w = np.zeros(27)
    opp = np.zeros(27, dtype=np.int32)
    ip = ctypes.POINTER(ctypes.c_int)
    Q = lib().oracle_lattice(LATTICES[lattice], c.ctypes.data_as(ip), _dp(w), opp.ctypes.data_as(ip),
                             h.ctypes.data_as(ip))
    return c[:3 * Q].reshape(Q, 3).copy(), w[:Q].copy(), opp[:Q].copy(), h[:3 * Q].reshape(Q, 3).copy()


def collide_node(lattice: str, reg: str, tau: float, f) -> np.ndarray:
    f = np.ascontiguousarray(f, dtype=np.float64)
    out = np.zeros_like(f)
    lib().oracle_collide_node(LATTICES[lattice], REGS[reg], float(tau), _dp(f), _dp(out))
    return out


def feq(lattice: str, rho: float, u) -> np.ndarray:
    Q = {"D2Q9": 9, "D3Q19": 19, "D3Q27": 27}[lattice]
    uu = np.zeros(3)
    uu[:len(u)] = u
    out = np.zeros(Q)
    lib().oracle_feq(LATTICES[lattice], float(rho), _dp(uu), _dp(out))
    return out


def aneq(idx, u, Pneq) -> float:
    idx = np.ascontiguousarray(idx, dtype=np.int32)
    u = np.ascontiguousarray(u, dtype=np.float64)
    P = np.ascontiguousarray(Pneq, dtype=np.float64).reshape(9)
    return lib().oracle_aneq(idx.ctypes.data_as(ctypes.POINTER(ctypes.c_int)), len(idx), _dp(u), _dp(P))


def M_of(lattice: str) -> int:
    return 6 if lattice == "D2Q9" else 10


def Q_of(lattice: str) -> int:
    return {"D2Q9": 9, "D3Q19": 19, "D3Q27": 27}[lattice]


class Oracle:
    """Distribution-form regularized LBM on a (nx, ny, nz) box.

    ``boundary`` maps face name ("x-", ...) to a dict with ``kind`` and
    optionally ``u`` (3-vector), ``rho`` and ``u_profile`` (array of shape
    [face nodes, D], row-major over the remaining axes, slower axis first).
    Missing faces are periodic.
    """

    def __init__(self, lattice, nx, ny, nz, tau, regularization, boundary=None, threads=1):
        self.lattice, self.reg = lattice, regularization
        self.D = 2 if lattice == "D2Q9" else 3
        self.shape = (nx, ny, 1 if self.D == 2 else nz)
        self.N = nx * ny * self.shape[2]
        # ABI array shape: [.][ny][nx] in 2D, [.][nz][ny][nx] in 3D
        self.grid = (ny, nx) if self.D == 2 else (nz, ny, nx)
        self.M, self.Q = M_of(lattice), Q_of(lattice)
        boundary = boundary or {}
        kind = np.zeros(6, dtype=np.int32)
        uw = np.zeros(18)
        rhow = np.ones(6)
        profs = (ctypes.POINTER(ctypes.c_double) * 6)()
        self._keep = []
        for F, name in enumerate(FACES):
            spec = boundary.get(name)
            if spec is None:
                continue
            kind[F] = BC[spec["kind"]]
            if "u" in spec:
                uu = np.zeros(3)
                uu[:len(spec["u"])] = spec["u"]
                uw[3 * F:3 * F + 3] = uu
            if "rho" in spec:
                rhow[F] = spec["rho"]
            if spec.get("u_profile") is not None:
                arr = np.ascontiguousarray(spec["u_profile"], dtype=np.float64).reshape(-1)
                self._keep.append(arr)
                profs[F] = _dp(arr)
        self._h = lib().oracle_create(LATTICES[lattice], nx, ny, self.shape[2], float(tau), REGS[regularization],
                                      kind.ctypes.data_as(ctypes.POINTER(ctypes.c_int)), _dp(uw), _dp(rhow),
                                      profs, int(threads))
        if not self._h:
            raise ValueError("oracle_create failed")

    def __del__(self):
        h = getattr(self, "_h", None)
        if h:
            lib().oracle_destroy(h)
            self._h = None

    def set_moments(self, m):
        m = np.ascontiguousarray(m, dtype=np.float64).reshape(self.M, self.N)
        lib().oracle_set_moments(self._h, _dp(m))

    def get_moments(self) -> np.ndarray:
        out = np.zeros((self.M, self.N))
        lib().oracle_get_moments(self._h, _dp(out))
        return out.reshape((self.M,) + self.grid)

    def set_f(self, f):
        f = np.ascontiguousarray(f, dtype=np.float64).reshape(self.Q, self.N)
        lib().oracle_set_f(self._h, _dp(f))

    def get_f(self) -> np.ndarray:
        out = np.zeros((self.Q, self.N))
        lib().oracle_get_f(self._h, _dp(out))
        return out.reshape((self.Q,) + self.grid)

    def get_populations(self) -> np.ndarray:
        out = np.zeros((self.Q, self.N))
        lib().oracle_get_populations(self._h, _dp(out))
        return out.reshape((self.Q,) + self.grid)

    def step(self, n=1):
        lib().oracle_step(self._h, int(n))
