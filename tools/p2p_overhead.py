"""Per-step cost of the slab decomposition on ONE GPU: a
D3Q19-R channel (fp64) of 1024 x 1024 x (128 P) as 1 rank vs P = 2 ranks of one
C5w slab (1024 x 1024 x 128) each, in one process, with the P2P transport (pushes fused into the boundary
launches, device counters, graph-replayed) and with the slab-group transport
(device-to-device ghost copies).  All ranks share the one GPU, so the total
work is equal and the difference is the decomposition's overhead: extra
launches, boundary-layer re-reads, waits/signals, pushes.  Prints one JSON line."""
import json
import sys
import time
from pathlib import Path

ROOT = Path(__file__).resolve().parents[1]
sys.path.insert(0, str(ROOT))

import torch  # noqa: E402

from paper_conf_sc_valero_laravgr23_b200 import configs, distributed, mrlbm  # noqa: E402


def timed(fn, syncs, reps=5):
    out = []
    for _ in range(reps):
        for s in syncs:
            s.sync()
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        fn()
        for s in syncs:
            s.sync()
        torch.cuda.synchronize()
        out.append(time.perf_counter() - t0)
    out.sort()
    return out[len(out) // 2]


def main(steps=128, P=2):
    c = configs.c5(nz=128 * P)
    m0 = c.initial_moments()
    args = (c.lattice, c.nx, c.ny, c.nz, c.tau, c.regularization, c.boundary)
    res = {"workload": f"D3Q19 recursive channel 1024x1024x{128 * P} fp64: 1 rank vs {P} ranks of 1024x1024x128",
           "steps": steps}
    with mrlbm.Solver(*args) as one:
        one.set_moments(m0)
        one.step(64)
        res["one_rank_ms_per_step"] = timed(lambda: one.step(steps), [one]) / steps * 1e3
    # P2P, P ranks in one process (own streams), batches replayed as graphs
    ranks = [mrlbm.Solver(*args, rank=r, nranks=P, transport="p2p") for r in range(P)]
    hs = [s.p2p_handle() for s in ranks]
    for s in ranks:
        distributed.p2p_connect(s, hs, False)
    for r, s in enumerate(ranks):
        s.set_moments(distributed.slab_of(m0, P, r))

    def run_p2p():
        for s in ranks:
            s.step(steps)
    run_p2p()
    res["p2p_2ranks_ms_per_step"] = timed(run_p2p, ranks) / steps * 1e3
    for s in ranks:
        s.close()
    # slab group (D2D copies), P ranks
    grp = [mrlbm.Solver(*args, rank=r, nranks=P) for r in range(P)]
    for r, s in enumerate(grp):
        s.set_moments(distributed.slab_of(m0, P, r))
    mrlbm.step_group(grp, 16)
    res["slab_group_2ranks_ms_per_step"] = timed(lambda: mrlbm.step_group(grp, steps), grp) / steps * 1e3
    for s in grp:
        s.close()
    base = res["one_rank_ms_per_step"]
    res["p2p_overhead_pct"] = 100.0 * (res["p2p_2ranks_ms_per_step"] / base - 1.0)
    res["slab_group_overhead_pct"] = 100.0 * (res["slab_group_2ranks_ms_per_step"] / base - 1.0)
    print(json.dumps(res), flush=True)


if __name__ == "__main__":
    main()
