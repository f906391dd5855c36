"""GPU parity of the finite-difference open faces (Latt et al. [6], the
paper's proxy-app inlet / outlet; R20, NEXT-3): the fused step plus the
face kernel, through the C ABI, against the oracle's FD faces."""
import numpy as np
import pytest

from parity import assert_parity, run_pair
from paper_conf_sc_valero_laravgr23_b200 import inputs

pytestmark = pytest.mark.gpu

VARIANTS = [(l, r) for l in ("D2Q9", "D3Q19", "D3Q27") for r in ("projective", "recursive")]


@pytest.mark.parametrize("precision", ["fp64", "fp32"])
@pytest.mark.parametrize("reg", ["projective", "recursive"])
def test_fd_poiseuille_channel_2d(reg, precision):
    """C1-shaped channel with FD inlet / outlet, 1000 steps from the analytic state."""
    nx, ny, U, tau = 128, 64, 0.05, 0.8
    prof = inputs.poiseuille_profile(ny, U)
    b = {"x-": {"kind": "velocity_fd", "u_profile": np.stack([prof, 0 * prof], 1)},
         "x+": {"kind": "pressure_fd", "rho": 1.0}, "y-": {"kind": "wall"}, "y+": {"kind": "wall"}}
    errs, got, _ = run_pair("D2Q9", reg, nx, ny, 1, tau, b, inputs.poiseuille_state(nx, ny, U, tau), 1000, precision)
    assert_parity(errs, precision, f"FD channel {reg}")
    assert np.abs(got[1] - prof[:, None]).max() / U < 5e-3


@pytest.mark.parametrize("lat,reg", VARIANTS)
def test_fd_random_odd_sizes(lat, reg):
    """Odd sizes spanning several tiles with ragged tails; smooth non-trivial
    state; FD faces on x (2D: periodic y; 3D: walls y, periodic z)."""
    D = 2 if lat == "D2Q9" else 3
    nx, ny, nz = (131, 67, 1) if D == 2 else (37, 29, 23)
    b = {"x-": {"kind": "velocity_fd", "u": [0.03, 0.01, 0.0]}, "x+": {"kind": "pressure_fd", "rho": 1.0}}
    if D == 3:
        b.update({"y-": {"kind": "wall"}, "y+": {"kind": "moving_wall", "u": [0.02, 0, 0.01]}})
    m0 = inputs.smooth_state(D, nx, ny, nz, U=0.03)
    errs, _, _ = run_pair(lat, reg, nx, ny, nz, 0.7, b, m0, 300 if D == 2 else 100)
    assert_parity(errs, "fp64", f"{lat}-{reg} FD x faces")


@pytest.mark.parametrize("precision", ["fp64", "fp32"])
@pytest.mark.parametrize("lat,reg", [("D3Q19", "recursive"), ("D3Q27", "recursive"), ("D3Q19", "projective")])
def test_fd_y_faces_3d(lat, reg, precision):
    """FD faces on y (kernel axis B) with periodic x (ghost columns) and walls on z."""
    nx, ny, nz = 35, 31, 19
    b = {"y-": {"kind": "velocity_fd", "u": [0.01, 0.02, 0.0]}, "y+": {"kind": "pressure_fd", "rho": 1.0},
         "z-": {"kind": "wall"}, "z+": {"kind": "wall"}}
    m0 = inputs.smooth_state(3, nx, ny, nz, U=0.03, seed=11)
    errs, _, _ = run_pair(lat, reg, nx, ny, nz, 0.7, b, m0, 100, precision)
    assert_parity(errs, precision, f"{lat}-{reg} FD y faces")
