"""Helpers shared by the GPU parity tests: run the CUDA path (through the
C-ABI binding) and the CPU oracle on the same seeded inputs and compare."""
import os

import numpy as np

THREADS = max(1, len(os.sched_getaffinity(0)))

# SURVEY 8(c) parity metric: per moment group, max|gpu - oracle| / max|oracle|
# (groups rho, u, Pi; pointwise relative error is undefined where u = 0).
# Thresholds from BASELINE.json north_star: 1e-11 fp64, 1e-4 fp32 (after 1000 steps).
TOL = {"fp64": 1e-11, "fp32": 1e-4}


def groups(D):
    return {"rho": [0], "u": list(range(1, 1 + D)), "Pi": list(range(1 + D, 6 if D == 2 else 10))}


def group_errors(gpu, ref, D):
    out = {}
    for g, idx in groups(D).items():
        den = np.abs(ref[idx]).max()
        den = den if den > 0 else 1.0
        out[g] = float(np.abs(gpu[idx] - ref[idx]).max() / den)
    return out


def group_scales(ref, D):
    """max|oracle| per group (the denominators of group_errors), for messages"""
    return {g: float(np.abs(ref[idx]).max()) for g, idx in groups(D).items()}


def run_pair(lat, reg, nx, ny, nz, tau, boundary, m0, steps, precision="fp64"):
    import oracle
    from paper_conf_sc_valero_laravgr23_b200 import mrlbm
    D = 2 if lat == "D2Q9" else 3
    o = oracle.Oracle(lat, nx, ny, nz, tau, reg, boundary, threads=THREADS)
    o.set_moments(m0)
    o.step(steps)
    ref = o.get_moments()
    with mrlbm.Solver(lat, nx, ny, nz, tau, reg, boundary, precision=precision) as s:
        s.set_moments(m0)
        s.step(steps)
        got = s.get_moments()
    return group_errors(got, ref, D), got, ref


def assert_parity(errs, precision, what=""):
    tol = TOL[precision]
    bad = {g: e for g, e in errs.items() if not (e <= tol)}
    assert not bad, f"{what}: parity errors {errs} exceed {tol}"
