"""Host-side checks that need no GPU: the C-ABI library loads and exports
every symbol include/mrlbm.h declares, argument validation, slab partition,
and the product path fails loudly (no CPU fallback) without a device."""
import os
import re
import sys
from pathlib import Path

import numpy as np
import pytest

from paper_conf_sc_valero_laravgr23_b200 import distributed, mrlbm

ROOT = Path(__file__).resolve().parents[1]


def header_symbols():
    txt = (ROOT / "include" / "mrlbm.h").read_text()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(mrlbm_[a-z_]+)\s*\(", txt)))


def test_library_exports_every_declared_symbol():
    syms = header_symbols()
    assert len(syms) >= 20
    for s in syms:
        assert hasattr(mrlbm.lib, s), s
    # the binding marshals every one of them
    assert set(syms) <= set(mrlbm.API) | set(mrlbm.HOST_HELPERS)


def test_library_is_built_for_sm100a():
    import subprocess
    out = subprocess.run(["cuobjdump", "-lelf", str(mrlbm._LIB_PATH)], capture_output=True, text=True).stdout
    assert "sm_100a" in out
    sass = subprocess.run(["cuobjdump", "-sass", str(mrlbm._LIB_PATH)], capture_output=True, text=True).stdout
    # the fused step kernels stage their tiles with TMA (UTMALDG) and mbarriers (SYNCS)
    assert "mrlbm_step_kernel" in sass and "UTMALDG" in sass and "SYNCS" in sass
    # the distribution-representation (ST) baseline kernels are in the same library
    assert "st_step_kernel" in sass


def test_status_strings():
    assert mrlbm.lib.mrlbm_status_string(0) == b"MRLBM_OK"
    assert mrlbm.lib.mrlbm_status_string(-7) == b"MRLBM_ERR_BUFFER_SIZE"


@pytest.mark.parametrize("n,p", [(10, 1), (10, 3), (1024, 8), (7, 7), (1000, 6)])
def test_partition_covers_axis(n, p):
    pieces = [mrlbm.partition(n, p, r) for r in range(p)]
    assert sum(nl for nl, _ in pieces) == n
    off = 0
    for r, (nl, o) in enumerate(pieces):
        assert o == off and nl >= n // p and nl <= n // p + 1
        assert (o, nl) == distributed.slab_bounds(n, p, r)
        off += nl


def walls(D):
    faces = ["x-", "x+", "y-", "y+"] + (["z-", "z+"] if D == 3 else [])
    return {f: {"kind": "wall"} for f in faces}


def test_validation_codes():
    INV, UNS = -1, -2
    assert mrlbm.validate("D3Q19", 8, 8, 8, 0.6) == 0
    assert mrlbm.validate("D3Q19", 8, 8, 8, 0.5) == INV            # tau <= 1/2 (eq 5)
    assert mrlbm.validate("D3Q19", 1, 8, 8, 0.6) == INV            # n < 2
    assert mrlbm.validate("D3Q27", 8, 8, 1, 0.6) == INV            # 3D needs nz >= 2
    assert mrlbm.validate("D2Q9", 8, 8, 1, 0.6, boundary={"x-": {"kind": "wall"}}) == INV  # one-sided periodic
    b = walls(3)
    b["y+"] = {"kind": "moving_wall", "u": [0.0, 0.1, 0.0]}       # normal lid velocity
    assert mrlbm.validate("D3Q19", 8, 8, 8, 0.6, boundary=b) == INV
    b = walls(3)
    b["z-"] = {"kind": "velocity", "u": [0, 0, 0.01]}              # open face on the sweep axis
    assert mrlbm.validate("D3Q19", 8, 8, 8, 0.6, boundary=b) == UNS
    b = walls(3)
    b["x-"] = {"kind": "velocity", "u": [0.01, 0, 0]}
    b["y+"] = {"kind": "pressure", "rho": 1.0}                      # open faces sharing an edge
    assert mrlbm.validate("D3Q19", 8, 8, 8, 0.6, boundary=b) == UNS
    b = walls(2)
    b["x-"] = {"kind": "velocity", "u": [0.01, 0, 0]}
    b["x+"] = {"kind": "pressure", "rho": 1.0}
    assert mrlbm.validate("D2Q9", 8, 8, 1, 0.6, boundary=b) == 0
    assert mrlbm.validate("D3Q19", 8, 8, 8, 0.6, nranks=8) == INV  # < 2 layers per rank


def test_validation_codes_distribution_representation():
    INV, UNS = -1, -2
    # BGK (Alg. 1) is not moment-closed: distributions only
    assert mrlbm.validate("D3Q19", 8, 8, 8, 0.6, "bgk") == UNS
    for reg in ("bgk", "projective", "recursive"):
        assert mrlbm.validate("D3Q19", 8, 8, 8, 0.6, reg, representation="distributions") == 0
    b = walls(3)
    b["y+"] = {"kind": "moving_wall", "u": [0.1, 0.0, 0.0]}
    assert mrlbm.validate("D2Q9", 8, 8, 1, 0.6, "bgk", boundary=walls(2), representation="distributions") == 0
    assert mrlbm.validate("D3Q27", 8, 8, 8, 0.6, "bgk", boundary=b, representation="distributions") == 0
    b = walls(2)
    b["x-"] = {"kind": "velocity", "u": [0.01, 0, 0]}
    b["x+"] = {"kind": "pressure", "rho": 1.0}
    assert mrlbm.validate("D2Q9", 8, 8, 1, 0.6, boundary=b, representation="distributions") == UNS
    assert mrlbm.validate("D3Q19", 8, 8, 8, 0.6, nranks=2, representation="distributions") == UNS
    assert mrlbm.validate("D3Q19", 8, 8, 8, 0.5, "bgk", representation="distributions") == INV


def test_validation_codes_fd_faces():
    """Finite-difference faces (R20): one rank, moments only, >= 3 nodes along bounded axes."""
    INV, UNS = -1, -2
    b = walls(2)
    b["x-"] = {"kind": "velocity_fd", "u": [0.01, 0, 0]}
    b["x+"] = {"kind": "pressure_fd", "rho": 1.0}
    assert mrlbm.validate("D2Q9", 8, 8, 1, 0.6, boundary=b) == 0
    assert mrlbm.validate("D2Q9", 2, 8, 1, 0.6, boundary=b) == INV          # 2 nodes along the normal
    assert mrlbm.validate("D2Q9", 8, 2, 1, 0.6, boundary=b) == INV          # 2 nodes along a walled tangent
    assert mrlbm.validate("D2Q9", 8, 8, 1, 0.6, boundary=b, nranks=2) == UNS
    assert mrlbm.validate("D2Q9", 8, 8, 1, 0.6, boundary=b, representation="distributions") == UNS
    b["x+"] = {"kind": "pressure_fd", "rho": 0.0}
    assert mrlbm.validate("D2Q9", 8, 8, 1, 0.6, boundary=b) == INV
    b = {"y-": {"kind": "velocity_fd", "u": [0, 0.01, 0]}, "y+": {"kind": "pressure", "rho": 1.0}}
    assert mrlbm.validate("D3Q19", 8, 8, 2, 0.6, boundary=b) == 0           # periodic x and z: no minimum
    assert mrlbm.validate("D3Q19", 8, 8, 8, 0.6, boundary={"z-": {"kind": "velocity_fd"}, "z+": {"kind": "wall"}}) == UNS


def test_create_fails_loudly_without_gpu():
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    with pytest.raises(mrlbm.MRLBMError) as e:
        mrlbm.Solver("D2Q9", 8, 8, 1, 0.6)
    assert e.value.status == -4  # MRLBM_ERR_CUDA: no silent CPU path


def test_slab_cut_and_reassemble():
    m = np.random.default_rng(0).standard_normal((10, 13, 5, 4))
    parts = [distributed.slab_of(m, 4, r) for r in range(4)]
    assert np.array_equal(np.concatenate(parts, axis=1), m)


def test_bench_workloads():
    """bench.py's workloads: C2 is BASELINE configs[1]; C5 runs as the C5w slab
    (1024 x 1024 x 128 per GPU) and grows along z with the ranks."""
    import bench
    c2 = bench.build_config("C2", "fp64", 1)
    assert (c2.lattice, c2.regularization, c2.nx, c2.ny, c2.precision) == ("D2Q9", "recursive", 4096, 4096, "fp64")
    assert bench.build_config("C2", "fp64", 4).ny == 4 * 4096
    for world in (1, 2, 8):
        c5 = bench.build_config("C5", "fp64", world)
        assert (c5.lattice, c5.regularization, c5.nx, c5.ny, c5.nz) == ("D3Q19", "recursive", 1024, 1024, 128 * world)
        assert c5.boundary["x-"]["u_profile"].shape == (128 * world, 1024, 3)
    assert "channel" in bench.workload_config(bench.build_config("C5", "fp64", 1), 1)["workload"]


def test_slab_neighbours_and_p2p_guards():
    from paper_conf_sc_valero_laravgr23_b200 import distributed
    assert distributed.slab_neighbours(4, 0, False) == (None, 1)
    assert distributed.slab_neighbours(4, 3, False) == (2, None)
    assert distributed.slab_neighbours(4, 0, True) == (3, 1)
    assert distributed.slab_neighbours(2, 1, True) == (0, 0)
    assert distributed.slab_axis_periodic({}, 3) and distributed.slab_axis_periodic({"x-": {"kind": "wall"}}, 2)
    assert not distributed.slab_axis_periodic({"z-": {"kind": "wall"}}, 3)
    assert mrlbm.TRANSPORTS == {"nccl": 0, "p2p": 1} and mrlbm.P2P_HANDLE_BYTES == 512


def test_bench_refuses_mismatched_world_size():
    """bench.py never prints a line whose rank count differs from --gpus."""
    import subprocess
    import sys
    env = dict(os.environ, WORLD_SIZE="2", RANK="0", LOCAL_RANK="0")
    r = subprocess.run([sys.executable, str(ROOT / "bench.py"), "--gpus", "1"], capture_output=True, text=True,
                       env=env, timeout=120)
    assert r.returncode == 2 and r.stdout.strip() == "", (r.returncode, r.stdout, r.stderr)


def test_bench_configs_weak_and_strong():
    sys.path.insert(0, str(ROOT))
    import bench
    c = bench.build_config("C5", "fp64", 8)
    assert (c.nx, c.ny, c.nz) == (1024, 1024, 1024) and c.nodes // 8 == 1024 * 1024 * 128
    c = bench.build_config("C5", "fp64", 1)
    assert (c.nx, c.ny, c.nz) == (1024, 1024, 128)
    c = bench.build_config("C5", "fp64", 4, strong=True)
    assert c.nz == 1024
    c = bench.build_config("C4", "fp32", 2, strong=True)
    assert (c.nx, c.ny, c.nz, c.precision) == (512, 512, 512, "fp32")
    c = bench.build_config("C2", "fp64", 1)
    assert (c.nx, c.ny, c.regularization) == (4096, 4096, "recursive")


def test_input_slabs_are_slices_of_the_global_field():
    """a rank's slab generated alone equals its slice of the global initial state"""
    from paper_conf_sc_valero_laravgr23_b200 import configs, inputs
    g = inputs.perturbed_rest(3, 21, 13, 17)
    for lo, hi in ((0, 5), (5, 11), (11, 17)):
        assert np.array_equal(inputs.perturbed_rest(3, 21, 13, 17, lo=lo, hi=hi, chunk=3), g[:, lo:hi])
    g2 = inputs.perturbed_rest(2, 19, 23)
    assert np.array_equal(inputs.perturbed_rest(2, 19, 23, lo=7, hi=16), g2[:, 7:16])
    c = configs.c5(nx=16, ny=12, nz=24)
    assert np.array_equal(c.initial_moments(lo=6, hi=12), c.initial_moments()[:, 6:12])
