"""P2P halo transport (options.transport = MRLBM_TRANSPORT_P2P): the fused step
stores its first / last layer straight into the neighbours' ghost planes
through peer memory and device-side counters order the steps.  P-rank results
must be BITWISE equal to the 1-rank run (same per-node arithmetic), both with
the ranks as handles of one process and as separate processes mapping each
other's buffers through CUDA IPC (all on device 0: gpurun has one GPU)."""
import multiprocessing as mp

import numpy as np
import pytest

from paper_conf_sc_valero_laravgr23_b200 import distributed, inputs

pytestmark = pytest.mark.gpu

CASES = [
    ("D3Q19", "recursive", (23, 17, 29), {"z-": {"kind": "wall"}, "z+": {"kind": "moving_wall", "u": [0.05, 0, 0]},
                                          "y-": {"kind": "wall"}, "y+": {"kind": "wall"}}, "fp64"),
    ("D3Q27", "projective", (19, 13, 21), {}, "fp64"),  # periodic z: rank 0 <-> rank P-1
    ("D3Q19", "projective", (31, 19, 24), {"x-": {"kind": "velocity", "u": [0.04, 0, 0]},
                                           "x+": {"kind": "pressure", "rho": 1.0},
                                           "y-": {"kind": "wall"}, "y+": {"kind": "wall"}}, "fp32"),
    ("D2Q9", "recursive", (70, 61, 1), {"x-": {"kind": "wall"}, "x+": {"kind": "wall"}, "y-": {"kind": "wall"},
                                        "y+": {"kind": "moving_wall", "u": [0.1, 0, 0]}}, "fp64"),
]
STEPS = 37


def reference(case):
    from paper_conf_sc_valero_laravgr23_b200 import mrlbm
    lat, reg, (nx, ny, nz), b, precision = case
    D = 2 if lat == "D2Q9" else 3
    with mrlbm.Solver(lat, nx, ny, nz, 0.7, reg, b, precision=precision) as one:
        one.set_moments(inputs.smooth_state(D, nx, ny, nz, U=0.05))
        one.step(STEPS)
        return one.get_moments()


@pytest.mark.parametrize("P", [2, 3])
@pytest.mark.parametrize("case", range(len(CASES)))
def test_p2p_in_process_bitwise(case, P):
    from paper_conf_sc_valero_laravgr23_b200 import mrlbm
    lat, reg, (nx, ny, nz), b, precision = CASES[case]
    D = 2 if lat == "D2Q9" else 3
    ref = reference(CASES[case])
    ranks = [mrlbm.Solver(lat, nx, ny, nz, 0.7, reg, b, precision=precision, rank=r, nranks=P, transport="p2p")
             for r in range(P)]
    try:
        handles = [s.p2p_handle() for s in ranks]
        for s in ranks:
            distributed.p2p_connect(s, handles, distributed.slab_axis_periodic(b, D))
        m0 = inputs.smooth_state(D, nx, ny, nz, U=0.05)
        for r, s in enumerate(ranks):
            s.set_moments(distributed.slab_of(m0, P, r))
        for _ in range(STEPS):   # each rank on its own stream; the device counters order them
            for s in ranks:
                s.step(1)
        for s in ranks:
            s.sync()
        got = np.concatenate([s.get_moments() for s in ranks], axis=1)
    finally:
        for s in ranks:
            s.close()
    assert np.array_equal(got, ref), f"max diff {np.abs(got - ref).max()}"


@pytest.mark.parametrize("case", [0, 3])
def test_p2p_in_process_graph_replay_bitwise(case):
    """P2P steps in batches (captured and replayed as CUDA graphs of 32 steps,
    each rank on its own stream, ordered only by the device counters)."""
    from paper_conf_sc_valero_laravgr23_b200 import mrlbm
    lat, reg, (nx, ny, nz), b, precision = CASES[case]
    D = 2 if lat == "D2Q9" else 3
    P, steps = 2, 70
    with mrlbm.Solver(lat, nx, ny, nz, 0.7, reg, b, precision=precision) as one:
        one.set_moments(inputs.smooth_state(D, nx, ny, nz, U=0.05))
        one.step(steps)
        ref = one.get_moments()
    ranks = [mrlbm.Solver(lat, nx, ny, nz, 0.7, reg, b, precision=precision, rank=r, nranks=P, transport="p2p")
             for r in range(P)]
    try:
        handles = [s.p2p_handle() for s in ranks]
        for s in ranks:
            distributed.p2p_connect(s, handles, distributed.slab_axis_periodic(b, D))
        m0 = inputs.smooth_state(D, nx, ny, nz, U=0.05)
        for r, s in enumerate(ranks):
            s.set_moments(distributed.slab_of(m0, P, r))
        for s in ranks:
            s.step(steps)   # 2 graph replays of 32 steps + 6 eager steps, enqueued rank after rank
        for s in ranks:
            s.sync()
        got = np.concatenate([s.get_moments() for s in ranks], axis=1)
    finally:
        for s in ranks:
            s.close()
    assert np.array_equal(got, ref), f"max diff {np.abs(got - ref).max()}"


def test_p2p_set_before_connect_is_refused():
    """The neighbours' ghost planes can only be filled once connected: setting
    the state of a P2P handle before mrlbm_p2p_connect is an error, not a
    silent zero halo."""
    from paper_conf_sc_valero_laravgr23_b200 import mrlbm
    nx, ny, nz = 19, 13, 12
    m0 = inputs.smooth_state(3, nx, ny, nz, U=0.05)
    ranks = [mrlbm.Solver("D3Q19", nx, ny, nz, 0.7, "projective", {}, rank=r, nranks=2, transport="p2p")
             for r in range(2)]
    try:
        with pytest.raises(mrlbm.MRLBMError, match="INVALID_ARGUMENT"):
            ranks[0].set_moments(distributed.slab_of(m0, 2, 0))
        with pytest.raises(mrlbm.MRLBMError, match="INVALID_ARGUMENT"):
            ranks[1].step(1)
    finally:
        for s in ranks:
            s.close()


@pytest.mark.parametrize("case", [0, 1])
def test_p2p_two_processes_ipc_bitwise(case):
    from p2p_worker import run_rank
    P = 2
    ctx = mp.get_context("spawn")
    pipes, procs = [], []
    for r in range(P):
        a, b_ = ctx.Pipe()
        p = ctx.Process(target=run_rank, args=(r, P, CASES[case], STEPS, b_), daemon=True)
        p.start()
        pipes.append(a)
        procs.append(p)
    try:
        def recv(c, tag):
            assert c.poll(300), f"rank timed out waiting for {tag}"
            t, v = c.recv()
            assert t == tag, f"rank reported {t}: {v}"
            return v
        handles = [recv(c, "handle") for c in pipes]
        for c in pipes:
            c.send(handles)
        for c in pipes:
            recv(c, "connected")
        for c in pipes:
            c.send("go")
        parts = [recv(c, "result") for c in pipes]
        for c in pipes:
            c.send("close")
    finally:
        for p in procs:
            p.join(timeout=60)
            if p.is_alive():
                p.kill()
    got = np.concatenate(parts, axis=1)
    ref = reference(CASES[case])
    assert np.array_equal(got, ref), f"max diff {np.abs(got - ref).max()}"
