"""Thin ctypes binding of libmrlbm.so (include/mrlbm.h) -- argument marshalling only.

Every step of the method runs in the library's CUDA kernels; this module
never computes any of it and has no CPU fallback: importing it without the
built library raises ImportError, and creating a solver without a CUDA
device fails with the library's MRLBM_ERR_CUDA.

    s = Solver("D3Q19", 64, 64, 64, tau=0.6, regularization="recursive",
               boundary={"z-": {"kind": "wall"}, ...}, precision="fp64")
    s.set_moments(m)            # [M][nz][ny][nx] fp64 (numpy) or device tensor
    s.step(100)
    m = s.get_moments()
"""
from __future__ import annotations

import ctypes
from pathlib import Path

import numpy as np

import os

# MRLBM_LIB: load another build of the same library (A/B performance comparisons)
_LIB_PATH = Path(os.environ.get("MRLBM_LIB") or Path(__file__).resolve().parent / "libmrlbm.so")

LATTICES = {"D2Q9": 0, "D3Q19": 1, "D3Q27": 2}
REGS = {"projective": 0, "recursive": 1, "bgk": 2}
REPRS = {"moments": 0, "distributions": 1}
PRECISIONS = {"fp64": 0, "fp32": 1}
TRANSPORTS = {"nccl": 0, "p2p": 1}
P2P_HANDLE_BYTES = 512  # MRLBM_P2P_HANDLE_BYTES
BC = {"periodic": 0, "wall": 1, "moving_wall": 2, "velocity": 3, "pressure": 4,
      "velocity_fd": 5, "pressure_fd": 6}
FACES = ("x-", "x+", "y-", "y+", "z-", "z+")
Q_OF = {"D2Q9": 9, "D3Q19": 19, "D3Q27": 27}
M_OF = {"D2Q9": 6, "D3Q19": 10, "D3Q27": 10}

# exported symbols of include/mrlbm.h (+ host-logic helpers of mrlbm.cu)
API = ("mrlbm_default_options", "mrlbm_create", "mrlbm_set_moments", "mrlbm_step", "mrlbm_get_moments",
       "mrlbm_get_populations", "mrlbm_set_moments_device", "mrlbm_get_moments_device", "mrlbm_sync",
       "mrlbm_check_finite", "mrlbm_query", "mrlbm_launch_count", "mrlbm_time_steps", "mrlbm_destroy",
       "mrlbm_status_string", "mrlbm_last_error", "mrlbm_nccl_unique_id", "mrlbm_set_populations",
       "mrlbm_p2p_handle", "mrlbm_p2p_connect", "mrlbm_comm_info")
HOST_HELPERS = ("mrlbm_partition", "mrlbm_validate", "mrlbm_validate_repr", "mrlbm_kernel_config", "mrlbm_step_group")


class Face(ctypes.Structure):
    _fields_ = [("kind", ctypes.c_int), ("u", ctypes.c_double * 3), ("rho", ctypes.c_double),
                ("u_profile", ctypes.POINTER(ctypes.c_double))]


class Boundary(ctypes.Structure):
    _fields_ = [("face", Face * 6)]


class Options(ctypes.Structure):
    _fields_ = [("precision", ctypes.c_int), ("device", ctypes.c_int), ("cuda_stream", ctypes.c_void_p),
                ("rank", ctypes.c_int), ("nranks", ctypes.c_int), ("nccl_unique_id", ctypes.c_void_p),
                ("representation", ctypes.c_int), ("transport", ctypes.c_int)]


def _load():
    if not _LIB_PATH.exists():
        raise ImportError(f"{_LIB_PATH} is not built; run `python -c 'import __graft_entry__ as g; g.build()'`")
    L = ctypes.CDLL(str(_LIB_PATH))
    i64, i64p, dp, vp = ctypes.c_int64, ctypes.POINTER(ctypes.c_int64), ctypes.POINTER(ctypes.c_double), ctypes.c_void_p
    ip = ctypes.POINTER(ctypes.c_int)
    sig = {
        "mrlbm_default_options": (None, [ctypes.POINTER(Options)]),
        "mrlbm_create": (ctypes.c_int, [ctypes.POINTER(vp), ctypes.c_int, i64, i64, i64, ctypes.c_double, ctypes.c_int,
                                        ctypes.POINTER(Boundary), ctypes.POINTER(Options)]),
        "mrlbm_set_moments": (ctypes.c_int, [vp, dp, i64]),
        "mrlbm_get_moments": (ctypes.c_int, [vp, dp, i64]),
        "mrlbm_get_populations": (ctypes.c_int, [vp, dp, i64]),
        "mrlbm_set_populations": (ctypes.c_int, [vp, dp, i64]),
        "mrlbm_set_moments_device": (ctypes.c_int, [vp, vp, i64]),
        "mrlbm_get_moments_device": (ctypes.c_int, [vp, vp, i64]),
        "mrlbm_step": (ctypes.c_int, [vp, i64]),
        "mrlbm_sync": (ctypes.c_int, [vp]),
        "mrlbm_check_finite": (ctypes.c_int, [vp]),
        "mrlbm_query": (ctypes.c_int, [vp, i64p, i64p, i64p, i64p, i64p]),
        "mrlbm_launch_count": (ctypes.c_int, [vp, i64p]),
        "mrlbm_time_steps": (ctypes.c_int, [vp, i64, dp]),
        "mrlbm_destroy": (None, [vp]),
        "mrlbm_status_string": (ctypes.c_char_p, [ctypes.c_int]),
        "mrlbm_last_error": (ctypes.c_char_p, []),
        "mrlbm_nccl_unique_id": (ctypes.c_int, [vp]),
        "mrlbm_partition": (ctypes.c_int, [i64, ctypes.c_int, ctypes.c_int, i64p, i64p]),
        "mrlbm_validate": (ctypes.c_int, [ctypes.c_int, i64, i64, i64, ctypes.c_double, ctypes.c_int,
                                          ctypes.POINTER(Boundary), ctypes.c_int]),
        "mrlbm_validate_repr": (ctypes.c_int, [ctypes.c_int, i64, i64, i64, ctypes.c_double, ctypes.c_int,
                                               ctypes.POINTER(Boundary), ctypes.c_int, ctypes.c_int]),
        "mrlbm_kernel_config": (ctypes.c_int, [vp, ip, ip, ip, ip, ip, ip, i64p]),
        "mrlbm_step_group": (ctypes.c_int, [ctypes.POINTER(vp), ctypes.c_int, i64]),
        "mrlbm_p2p_handle": (ctypes.c_int, [vp, vp]),
        "mrlbm_p2p_connect": (ctypes.c_int, [vp, vp, vp]),
        "mrlbm_comm_info": (ctypes.c_int, [vp, ip, ip, ip]),
    }
    for name, (res, args) in sig.items():
        if not hasattr(L, name) and os.environ.get("MRLBM_LIB"):
            continue  # an older build loaded for an A/B timing comparison
        fn = getattr(L, name)
        fn.restype = res
        fn.argtypes = args
    return L


lib = _load()


class MRLBMError(RuntimeError):
    def __init__(self, status, where):
        self.status = status
        msg = lib.mrlbm_status_string(status).decode()
        detail = lib.mrlbm_last_error().decode()
        super().__init__(f"{where}: {msg} ({detail})")


def _check(status, where):
    if status != 0:
        raise MRLBMError(status, where)


def make_boundary(boundary, D, keep):
    """dict face-name -> spec  ->  mrlbm_boundary (missing faces periodic)."""
    b = Boundary()
    for F, name in enumerate(FACES):
        spec = (boundary or {}).get(name)
        f = b.face[F]
        f.kind = 0
        f.rho = 1.0
        if spec is None:
            continue
        f.kind = BC[spec["kind"]]
        u = list(spec.get("u", [0.0, 0.0, 0.0])) + [0.0] * 3
        for q in range(3):
            f.u[q] = float(u[q])
        f.rho = float(spec.get("rho", 1.0))
        prof = spec.get("u_profile")
        if prof is not None:
            arr = np.ascontiguousarray(prof, dtype=np.float64).reshape(-1)
            keep.append(arr)
            f.u_profile = arr.ctypes.data_as(ctypes.POINTER(ctypes.c_double))
    return b


def partition(n, nranks, rank):
    """(n_local, offset) of the library's slab partition (host arithmetic only)."""
    nl, off = ctypes.c_int64(), ctypes.c_int64()
    _check(lib.mrlbm_partition(n, nranks, rank, ctypes.byref(nl), ctypes.byref(off)), "mrlbm_partition")
    return nl.value, off.value


def validate(lattice, nx, ny, nz, tau, regularization="projective", boundary=None, nranks=1,
             representation="moments"):
    """Status mrlbm_create would return for these arguments (no GPU needed)."""
    keep = []
    D = 2 if lattice == "D2Q9" else 3
    b = make_boundary(boundary, D, keep)
    return lib.mrlbm_validate_repr(LATTICES[lattice], nx, ny, nz if D == 3 else 1, float(tau), REGS[regularization],
                                   ctypes.byref(b), nranks, REPRS[representation])


def step_group(solvers, n):
    """Advance a single-process slab group (ranks 0..P-1 created without an NCCL id)."""
    arr = (ctypes.c_void_p * len(solvers))(*[s._h.value for s in solvers])
    _check(lib.mrlbm_step_group(arr, len(solvers), int(n)), "mrlbm_step_group")


def nccl_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(128)
    _check(lib.mrlbm_nccl_unique_id(buf), "mrlbm_nccl_unique_id")
    return buf.raw


class Solver:
    """One mrlbm_t handle (see include/mrlbm.h for the semantics)."""

    def __init__(self, lattice, nx, ny, nz=1, tau=0.6, regularization="projective", boundary=None,
                 precision="fp64", device=-1, stream=None, rank=0, nranks=1, nccl_id: bytes | None = None,
                 representation="moments", transport="nccl"):
        self.lattice, self.regularization, self.precision = lattice, regularization, precision
        self.representation = representation
        self.rank, self.nranks = rank, nranks
        self.D = 2 if lattice == "D2Q9" else 3
        self.M, self.Q = M_OF[lattice], Q_OF[lattice]
        self.nx, self.ny, self.nz = nx, ny, (nz if self.D == 3 else 1)
        self._keep = []
        b = make_boundary(boundary, self.D, self._keep)
        o = Options()
        lib.mrlbm_default_options(ctypes.byref(o))
        o.precision = PRECISIONS[precision]
        o.device = device
        o.cuda_stream = stream
        o.rank, o.nranks = rank, nranks
        o.representation = REPRS[representation]
        o.transport = TRANSPORTS[transport]
        if nccl_id is not None:
            self._id = ctypes.create_string_buffer(bytes(nccl_id), 128)
            o.nccl_unique_id = ctypes.cast(self._id, ctypes.c_void_p)
        h = ctypes.c_void_p()
        _check(lib.mrlbm_create(ctypes.byref(h), LATTICES[lattice], nx, ny, self.nz, float(tau),
                                REGS[regularization], ctypes.byref(b), ctypes.byref(o)), "mrlbm_create")
        self._h = h
        M, Q, nl, off, by = (ctypes.c_int64() for _ in range(5))
        _check(lib.mrlbm_query(h, *(ctypes.byref(v) for v in (M, Q, nl, off, by))), "mrlbm_query")
        self.n_local, self.offset, self.device_bytes = nl.value, off.value, by.value
        self.grid = (self.n_local, nx) if self.D == 2 else (self.n_local, ny, nx)
        self.N = int(np.prod(self.grid))

    def close(self):
        if getattr(self, "_h", None):
            lib.mrlbm_destroy(self._h)
            self._h = None

    def __del__(self):
        self.close()

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()

    # ---- host I/O (fp64, ABI layout)
    def set_moments(self, m):
        if hasattr(m, "data_ptr") and getattr(m, "is_cuda", False):
            return self.set_moments_device(m)
        a = np.ascontiguousarray(m, dtype=np.float64)
        _check(lib.mrlbm_set_moments(self._h, a.ctypes.data_as(ctypes.POINTER(ctypes.c_double)), a.size),
               "mrlbm_set_moments")

    def get_moments(self) -> np.ndarray:
        out = np.empty((self.M,) + self.grid, dtype=np.float64)
        _check(lib.mrlbm_get_moments(self._h, out.ctypes.data_as(ctypes.POINTER(ctypes.c_double)), out.size),
               "mrlbm_get_moments")
        return out

    def get_populations(self) -> np.ndarray:
        out = np.empty((self.Q,) + self.grid, dtype=np.float64)
        _check(lib.mrlbm_get_populations(self._h, out.ctypes.data_as(ctypes.POINTER(ctypes.c_double)), out.size),
               "mrlbm_get_populations")
        return out

    def set_populations(self, f):
        """pre-collision populations [Q][...] (fp64): stored as is (distributions)
        or as their moments (moments representation)."""
        a = np.ascontiguousarray(f, dtype=np.float64)
        _check(lib.mrlbm_set_populations(self._h, a.ctypes.data_as(ctypes.POINTER(ctypes.c_double)), a.size),
               "mrlbm_set_populations")

    # ---- device I/O (torch fp64 CUDA tensors in the ABI layout)
    # The library copies on its own stream and returns when the copy is done;
    # the tensor's producer on torch's current stream must be finished first.
    def set_moments_device(self, t):
        import torch
        assert t.is_contiguous() and t.dtype == torch.float64 and t.is_cuda
        torch.cuda.current_stream(t.device).synchronize()
        _check(lib.mrlbm_set_moments_device(self._h, ctypes.c_void_p(t.data_ptr()), t.numel()),
               "mrlbm_set_moments_device")

    def get_moments_device(self, t):
        import torch
        assert t.is_contiguous() and t.dtype == torch.float64 and t.is_cuda
        # t must not be in use by torch's stream while the library writes it
        torch.cuda.current_stream(t.device).synchronize()
        _check(lib.mrlbm_get_moments_device(self._h, ctypes.c_void_p(t.data_ptr()), t.numel()),
               "mrlbm_get_moments_device")

    def step(self, n=1):
        _check(lib.mrlbm_step(self._h, int(n)), "mrlbm_step")

    # ---- P2P transport (transport="p2p", nranks > 1)
    def p2p_handle(self) -> bytes:
        buf = ctypes.create_string_buffer(P2P_HANDLE_BYTES)
        _check(lib.mrlbm_p2p_handle(self._h, ctypes.cast(buf, ctypes.c_void_p)), "mrlbm_p2p_handle")
        return buf.raw

    def p2p_connect(self, lo: bytes | None, hi: bytes | None):
        """map the lower / upper neighbour's handle (None where the slab has none)"""
        bl = ctypes.create_string_buffer(bytes(lo), P2P_HANDLE_BYTES) if lo is not None else None
        bh = ctypes.create_string_buffer(bytes(hi), P2P_HANDLE_BYTES) if hi is not None else None
        self._p2p_keep = (bl, bh)
        _check(lib.mrlbm_p2p_connect(self._h, ctypes.cast(bl, ctypes.c_void_p) if bl is not None else None,
                                     ctypes.cast(bh, ctypes.c_void_p) if bh is not None else None),
               "mrlbm_p2p_connect")

    def sync(self):
        _check(lib.mrlbm_sync(self._h), "mrlbm_sync")

    def check_finite(self):
        _check(lib.mrlbm_check_finite(self._h), "mrlbm_check_finite")

    def comm_info(self) -> dict:
        """halo transport and the communicator's own view of the rank count"""
        t, n, r = ctypes.c_int(), ctypes.c_int(), ctypes.c_int()
        _check(lib.mrlbm_comm_info(self._h, ctypes.byref(t), ctypes.byref(n), ctypes.byref(r)), "mrlbm_comm_info")
        return {"transport": ["single", "nccl", "p2p", "slab_group"][t.value], "comm_nranks": n.value,
                "comm_rank": r.value}

    def launch_count(self) -> int:
        k = ctypes.c_int64()
        _check(lib.mrlbm_launch_count(self._h, ctypes.byref(k)), "mrlbm_launch_count")
        return k.value

    def time_steps(self, n) -> float:
        ms = ctypes.c_double()
        _check(lib.mrlbm_time_steps(self._h, int(n), ctypes.byref(ms)), "mrlbm_time_steps")
        return ms.value

    def kernel_config(self) -> dict:
        v = [ctypes.c_int() for _ in range(6)]
        sm = ctypes.c_int64()
        _check(lib.mrlbm_kernel_config(self._h, *(ctypes.byref(x) for x in v), ctypes.byref(sm)),
               "mrlbm_kernel_config")
        keys = ("TA", "TB", "S", "seg_len", "grid_x", "grid_y")
        d = {k: x.value for k, x in zip(keys, v)}
        d["smem_bytes"] = sm.value
        return d
