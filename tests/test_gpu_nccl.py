"""The NCCL halo transport on real GPUs (one rank per GPU under torchrun),
bitwise against the 1-rank run.  Needs >= 2 visible GPUs: skipped on the
1-GPU test box (the decomposition itself is verified on one GPU by the
slab-group and P2P tests)."""
import os
import socket
import subprocess
import sys
from pathlib import Path

import pytest

pytestmark = pytest.mark.gpu
HERE = Path(__file__).resolve().parent


def _ngpus():
    import torch
    return torch.cuda.device_count() if torch.cuda.is_available() else 0


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


@pytest.mark.skipif(_ngpus() < 2, reason="needs >= 2 GPUs (one NCCL rank per GPU)")
@pytest.mark.parametrize("case", ["walled", "periodic", "channel_fp32"])
def test_nccl_transport_bitwise(case):
    n = min(_ngpus(), 4)
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}",
           "--master-addr", "127.0.0.1", "--master-port", str(_free_port()), str(HERE / "nccl_worker.py"), case]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=600, env=dict(os.environ, NCCL_DEBUG="WARN"))
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-3000:]
    assert f"NCCL_PARITY {case} world={n} bitwise=True" in r.stdout
