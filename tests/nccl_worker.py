"""torchrun worker for tests/test_gpu_nccl.py: one rank per GPU, the library's
NCCL halo transport (options.nccl_unique_id), compared BITWISE with a 1-rank run.
Host plumbing (ncclUniqueId broadcast, slab gather) goes through gloo."""
import os
import sys
from pathlib import Path

ROOT = Path(__file__).resolve().parents[1]
sys.path.insert(0, str(ROOT))

import numpy as np  # noqa: E402
import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402

from paper_conf_sc_valero_laravgr23_b200 import distributed, inputs, mrlbm  # noqa: E402

CASES = {
    "walled": ("D3Q19", "recursive", (37, 23, 41), {"z-": {"kind": "wall"}, "z+": {"kind": "moving_wall", "u": [0.05, 0, 0]},
                                                   "y-": {"kind": "wall"}, "y+": {"kind": "wall"}}, "fp64"),
    "periodic": ("D3Q27", "projective", (29, 17, 40), {}, "fp64"),
    "channel_fp32": ("D3Q19", "projective", (33, 19, 36), {"x-": {"kind": "velocity", "u": [0.04, 0, 0]},
                                                          "x+": {"kind": "pressure", "rho": 1.0},
                                                          "y-": {"kind": "wall"}, "y+": {"kind": "wall"}}, "fp32"),
}
STEPS = 41


def main():
    name = sys.argv[1]
    lat, reg, (nx, ny, nz), b, precision = CASES[name]
    dist.init_process_group("gloo")
    rank, world = dist.get_rank(), dist.get_world_size()
    local = int(os.environ.get("LOCAL_RANK", rank))
    torch.cuda.set_device(local)
    ids = [mrlbm.nccl_unique_id() if rank == 0 else None]
    dist.broadcast_object_list(ids, 0)
    m0 = inputs.smooth_state(3, nx, ny, nz, U=0.05)
    with mrlbm.Solver(lat, nx, ny, nz, 0.7, reg, b, precision=precision, device=local, rank=rank, nranks=world,
                      nccl_id=ids[0]) as s:
        info = s.comm_info()
        assert info["transport"] == "nccl" and info["comm_nranks"] == world and info["comm_rank"] == rank, info
        s.set_moments(distributed.slab_of(m0, world, rank))
        s.step(STEPS)          # graph-free multi-rank steps
        s.sync()
        got = distributed.gather_slabs(s.get_moments(), nz)
    if rank == 0:
        with mrlbm.Solver(lat, nx, ny, nz, 0.7, reg, b, precision=precision, device=local) as one:
            one.set_moments(m0)
            one.step(STEPS)
            ref = one.get_moments()
        ok = np.array_equal(got, ref)
        print(f"NCCL_PARITY {name} world={world} bitwise={ok} maxdiff={np.abs(got - ref).max():.3e}", flush=True)
        if not ok:
            sys.exit(1)
    dist.barrier()
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
