"""World-size-2 gloo tests (CPU) of the multi-GPU host logic: ncclUniqueId
bootstrap broadcast, slab partition agreement across ranks, slab gather."""
import os
import socket
import sys
from pathlib import Path

import numpy as np
import pytest

ROOT = Path(__file__).resolve().parents[1]


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    sys.path.insert(0, str(ROOT))
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    import torch
    import torch.distributed as dist
    from paper_conf_sc_valero_laravgr23_b200 import distributed, inputs, mrlbm
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        # 1) ncclUniqueId created on rank 0, broadcast out of band (as bench.py does)
        idt = torch.zeros(128, dtype=torch.uint8)
        if rank == 0:
            idt.copy_(torch.frombuffer(bytearray(mrlbm.nccl_unique_id()), dtype=torch.uint8))
        dist.broadcast(idt, 0)
        ids = [torch.zeros(128, dtype=torch.uint8) for _ in range(world)]
        dist.all_gather(ids, idt)
        same_id = all(torch.equal(ids[0], x) for x in ids)
        # 2) every rank derives the same partition from the C library
        nz = 37
        nl, off = mrlbm.partition(nz, world, rank)
        parts = [torch.zeros(2, dtype=torch.int64) for _ in range(world)]
        dist.all_gather(parts, torch.tensor([nl, off]))
        parts = [tuple(p.tolist()) for p in parts]
        # 3) slabs of a global field gather back to the global field
        m = inputs.perturbed_rest(3, 6, 5, nz)
        local = distributed.slab_of(m, world, rank)
        assert local.shape[1] == nl
        full = distributed.gather_slabs(local, nz)
        q.put((rank, same_id, parts, bool(np.array_equal(full, m))))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2])
def test_gloo_slab_bootstrap(world):
    import multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=180) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for rank, same_id, parts, ok in res:
        assert same_id
        assert sum(n for n, _ in parts) == 37 and parts[0][1] == 0 and parts[1][1] == parts[0][0]
        assert ok
