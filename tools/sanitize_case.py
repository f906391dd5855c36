"""Small cases of the fused step for compute-sanitizer (tools/sanitize.sh):
2D and 3D, walls + lid, open faces, periodic, a P2P pair in one process, and
(3D) the cluster variant.  A few steps each; exits non-zero on a library error."""
import os
import sys
from pathlib import Path

ROOT = Path(__file__).resolve().parents[1]
sys.path.insert(0, str(ROOT))

from paper_conf_sc_valero_laravgr23_b200 import distributed, inputs, mrlbm  # noqa: E402


def run(lat, reg, prec, n, b, steps=6):
    D = 2 if lat == "D2Q9" else 3
    m0 = inputs.smooth_state(D, *n, U=0.05)
    with mrlbm.Solver(lat, *n, 0.7, reg, b, precision=prec) as s:
        s.set_moments(m0)
        s.step(steps)
        s.get_moments()
        s.get_populations()
    print(f"ok {lat}-{reg}-{prec} {n} {sorted(b)} cluster={os.environ.get('MRLBM_CLUSTER', 'default')}", flush=True)


def p2p_pair():
    lat, n = "D3Q19", (23, 17, 12)
    b = {"z-": {"kind": "wall"}, "z+": {"kind": "moving_wall", "u": [0.05, 0, 0]}}
    m0 = inputs.smooth_state(3, *n, U=0.05)
    ranks = [mrlbm.Solver(lat, *n, 0.7, "recursive", b, rank=r, nranks=2, transport="p2p") for r in range(2)]
    try:
        hs = [s.p2p_handle() for s in ranks]
        for s in ranks:
            distributed.p2p_connect(s, hs, False)
        for r, s in enumerate(ranks):
            s.set_moments(distributed.slab_of(m0, 2, r))
        for _ in range(4):
            for s in ranks:
                s.step(1)
        for s in ranks:
            s.sync()
    finally:
        for s in ranks:
            s.close()
    print("ok P2P pair in one process", flush=True)


if __name__ == "__main__":
    which = sys.argv[1] if len(sys.argv) > 1 else "all"
    walls2 = {"x-": {"kind": "wall"}, "x+": {"kind": "wall"}, "y-": {"kind": "wall"},
              "y+": {"kind": "moving_wall", "u": [0.1, 0, 0]}}
    chan3 = {"x-": {"kind": "velocity", "u": [0.04, 0, 0]}, "x+": {"kind": "pressure", "rho": 1.0},
             "y-": {"kind": "wall"}, "y+": {"kind": "wall"}, "z-": {"kind": "wall"}, "z+": {"kind": "wall"}}
    if which in ("all", "2d"):
        run("D2Q9", "recursive", "fp64", (131, 40, 1), walls2)
        run("D2Q9", "projective", "fp32", (131, 40, 1), {})
    if which in ("all", "3d"):
        run("D3Q19", "recursive", "fp64", (37, 29, 11), chan3)
        run("D3Q19", "projective", "fp64", (33, 15, 9), {})
        run("D3Q27", "recursive", "fp32", (33, 31, 9), {"y+": {"kind": "moving_wall", "u": [0.1, 0, 0]},
                                                      "y-": {"kind": "wall"}})
        # round 3: the paired kernel for D3Q19 fp32 and the product-form D3Q27-R fp64
        run("D3Q19", "recursive", "fp32", (37, 29, 11), chan3)
        run("D3Q27", "recursive", "fp64", (33, 19, 9), chan3)
    if which in ("all", "p2p"):
        p2p_pair()
