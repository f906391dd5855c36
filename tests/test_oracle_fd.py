"""Pins of the oracle's finite-difference open faces (Latt et al. [6], the
scheme of the paper's proxy apps, "finite difference boundary
conditions at the inlet and outlet [6]"; R20).

The FD face keeps the regularized face's rho / u rule and sets the
non-equilibrium stress to the Chapman-Enskog value of the new velocity field,
Pi^neq = -rho tau c_s^2 (grad u + grad u^T), with second-order differences.
Pinned against
  * numpy.gradient(edge_order=2) -- the library's second-order central /
    one-sided stencils -- applied to the oracle's own post-step velocity field
    (np.roll central differences on periodic axes);
  * the closed-form stress of the Poiseuille parabola at the inlet;
  * the analytic Poiseuille solution (accuracy, second-order convergence) and
    the prescribed outlet density.
"""
import numpy as np
import pytest

from paper_conf_sc_valero_laravgr23_b200 import inputs

CS2 = 1.0 / 3.0


def _grad(u, axis, periodic):
    """d u / d axis with unit spacing: central (wrapped when periodic), else
    numpy's second-order one-sided stencils at the two ends."""
    if periodic:
        return 0.5 * (np.roll(u, -1, axis) - np.roll(u, 1, axis))
    return np.gradient(u, axis=axis, edge_order=2)


def _check_fd_face_stress(mm, tau, D, face_axis, periodic_axes, faces=(0, -1)):
    """Pi - rho u u at the face nodes equals -rho tau c_s^2 (g + g^T) from the
    library gradient of the whole post-step velocity field."""
    rho = mm[0]
    u = [mm[1 + a] for a in range(D)]
    # array axes: 2D [y][x], 3D [z][y][x] -> physical axis a is array axis D-1-a
    g = [[_grad(u[b], D - 1 - a, a in periodic_axes) for b in range(D)] for a in range(D)]
    slot = {(0, 0): 3, (1, 1): 4, (0, 1): 5} if D == 2 else \
        {(0, 0): 4, (1, 1): 5, (2, 2): 6, (0, 1): 7, (0, 2): 8, (1, 2): 9}
    worst = 0.0
    for (a, b), s in slot.items():
        pneq = mm[s] - rho * u[a] * u[b]
        want = -rho * tau * CS2 * (g[a][b] + g[b][a])
        ax = D - 1 - face_axis
        for idx in faces:
            sl = [slice(None)] * D
            sl[ax] = idx
            sl = tuple(sl)
            scale = max(np.abs(want).max(), 1e-30)
            worst = max(worst, np.abs(pneq[sl] - want[sl]).max() / scale)
    return worst


def _channel2d(ny, nx, U, tau, kind="fd"):
    prof = inputs.poiseuille_profile(ny, U)
    up = np.stack([prof, 0 * prof], 1)
    suffix = "_fd" if kind == "fd" else ""
    return {"x-": {"kind": "velocity" + suffix, "u_profile": up}, "x+": {"kind": "pressure" + suffix, "rho": 1.0},
            "y-": {"kind": "wall"}, "y+": {"kind": "wall"}}, prof


@pytest.mark.parametrize("reg", ["projective", "recursive"])
def test_fd_stress_matches_library_gradient_2d(oracle_mod, reg):
    ny, nx, U, tau = 11, 13, 0.05, 0.8
    b, _ = _channel2d(ny, nx, U, tau)
    o = oracle_mod.Oracle("D2Q9", nx, ny, 1, tau, reg, b)
    o.set_moments(inputs.smooth_state(2, nx, ny, 1, U=U, seed=3))
    o.step(3)
    mm = o.get_moments()
    assert _check_fd_face_stress(mm, tau, 2, face_axis=0, periodic_axes=()) < 1e-12


@pytest.mark.parametrize("lat,reg", [("D3Q19", "projective"), ("D3Q19", "recursive"), ("D3Q27", "recursive")])
def test_fd_stress_matches_library_gradient_3d(oracle_mod, lat, reg):
    """3D: FD faces on y (velocity, uniform u) and x walls, z periodic: the
    tangential derivatives along x use one-sided stencils at the wall edges,
    along z the wrapped central difference."""
    nx, ny, nz, tau = 7, 9, 6, 0.7
    b = {"x-": {"kind": "wall"}, "x+": {"kind": "wall"},
         "y-": {"kind": "velocity_fd", "u": [0.0, 0.02, 0.0]}, "y+": {"kind": "pressure_fd", "rho": 1.0}}
    o = oracle_mod.Oracle(lat, nx, ny, nz, tau, reg, b)
    o.set_moments(inputs.smooth_state(3, nx, ny, nz, U=0.03, seed=5))
    o.step(2)
    mm = o.get_moments()
    assert _check_fd_face_stress(mm, tau, 3, face_axis=1, periodic_axes=(2,)) < 1e-12
    # the prescribed face values
    assert np.allclose(mm[2][:, 0, :], 0.02, atol=1e-13) and np.allclose(mm[0][:, -1, :], 1.0, atol=1e-13)


def test_fd_inlet_stress_closed_form(oracle_mod):
    """Poiseuille inlet: u_x is the prescribed parabola on the face, so the
    tangential derivative is exact and Pi^neq_xy = -rho tau c_s^2 du_x/dy of the
    parabola (the interior enters only through d u_y/dx, ~0)."""
    ny, nx, U, tau = 16, 32, 0.05, 0.8
    b, prof = _channel2d(ny, nx, U, tau)
    o = oracle_mod.Oracle("D2Q9", nx, ny, 1, tau, "projective", b)
    o.set_moments(inputs.poiseuille_state(nx, ny, U, tau))
    o.step(1)
    mm = o.get_moments()
    yc = np.arange(ny) + 0.5
    duy = 4.0 * U * (ny - 2 * yc) / ny ** 2
    pneq_xy = mm[5][:, 0] - mm[0][:, 0] * mm[1][:, 0] * mm[2][:, 0]
    want = -mm[0][:, 0] * tau * CS2 * duy
    assert np.abs(pneq_xy - want).max() / np.abs(want).max() < 1e-3
    assert np.allclose(mm[1][:, 0], prof, atol=1e-15)


@pytest.mark.parametrize("reg", ["projective", "recursive"])
def test_fd_poiseuille_accuracy(oracle_mod, reg):
    """The FD channel keeps the analytic Poiseuille state (5e-3 U at H = 64
    after 1000 steps), converges at second order, holds the outlet density."""
    errs = []
    for ny in (16, 32, 64):
        nx = 2 * ny
        tau, U = 0.8, 0.05
        b, prof = _channel2d(ny, nx, U, tau)
        o = oracle_mod.Oracle("D2Q9", nx, ny, 1, tau, reg, b, threads=4)
        o.set_moments(inputs.poiseuille_state(nx, ny, U, tau))
        o.step(1000)
        mm = o.get_moments()
        errs.append(np.abs(mm[1] - prof[:, None]).max() / U)
    assert errs[2] < 5e-3
    assert errs[0] / errs[1] > 2.0 and errs[1] / errs[2] > 2.0
    assert np.allclose(mm[0][:, -1], 1.0, atol=1e-12)


def test_fd_differs_from_regularized_only_on_the_faces(oracle_mod):
    """One step from the same state: FD and regularized faces agree on rho, u
    everywhere and on Pi away from the open faces."""
    ny, nx, U, tau = 12, 14, 0.05, 0.8
    out = {}
    for kind in ("fd", "reg"):
        b, _ = _channel2d(ny, nx, U, tau, kind)
        o = oracle_mod.Oracle("D2Q9", nx, ny, 1, tau, "recursive", b)
        o.set_moments(inputs.smooth_state(2, nx, ny, 1, U=0.05, seed=9))
        o.step(1)
        out[kind] = o.get_moments()
    a, r = out["fd"], out["reg"]
    assert np.abs(a[:3] - r[:3]).max() < 1e-15
    assert np.abs(a[3:, :, 1:-1] - r[3:, :, 1:-1]).max() < 1e-15
    assert np.abs(a[3:, :, 0] - r[3:, :, 0]).max() > 1e-8
