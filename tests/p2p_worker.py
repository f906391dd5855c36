"""Worker of the two-process P2P-transport test (tests/test_gpu_p2p.py): one
rank of a z-slab decomposition in its own process, its peer's state buffers
mapped through CUDA IPC (both ranks on device 0; across GPUs the same stores
go over NVLink).  Handles are exchanged through multiprocessing pipes."""
import sys
from pathlib import Path

ROOT = Path(__file__).resolve().parents[1]
sys.path.insert(0, str(ROOT))


def run_rank(rank, nranks, case, steps, conn):
    import numpy as np
    from paper_conf_sc_valero_laravgr23_b200 import distributed, inputs, mrlbm
    lat, reg, (nx, ny, nz), b, precision = case
    D = 2 if lat == "D2Q9" else 3
    try:
        s = mrlbm.Solver(lat, nx, ny, nz, 0.7, reg, b, precision=precision, device=0, rank=rank, nranks=nranks,
                         transport="p2p")
        conn.send(("handle", s.p2p_handle()))
        handles = conn.recv()
        distributed.p2p_connect(s, handles, distributed.slab_axis_periodic(b, D))
        conn.send(("connected", None))
        assert conn.recv() == "go"
        m0 = inputs.smooth_state(D, nx, ny, nz, U=0.05)
        s.set_moments(distributed.slab_of(m0, nranks, rank))
        s.step(steps)
        s.sync()
        conn.send(("result", s.get_moments()))
        assert conn.recv() == "close"
        s.close()
    except Exception as e:  # report instead of hanging the parent
        conn.send(("error", repr(e)))
