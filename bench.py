"""bench.py -- MR-LBM throughput on B200 (BASELINE.json metric: MLUPS per GPU
and whole box; achieved HBM GB/s vs peak).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config C2] [--precision fp64]
  python bench.py --impl reference ...      # the CPU oracle arm (bounded sample)
  python bench.py --method ST [--collision bgk] ...  # the paper's ST baseline on the GPU

A "step" is one timestep of the whole hot path (load moments -> collide ->
reconstruct -> stream -> boundaries -> moments -> store; SURVEY 8(a) rows
a1-a9) over the whole domain.  Default workload = BASELINE.json configs[1]
(C2: D2Q9 recursive-regularized lid-driven cavity 4096^2, fp64, 1 B200).
For N > 1 (torchrun) every rank owns one 4096 x 4096 y-slab of a 4096 x
4096N cavity (weak scaling) and exchanges one boundary row of moments per
step with its neighbours over NCCL.

--method ST runs the same workload in the paper's standard distribution
representation (Alg. 1: two Q-population lattices, 2 Q w bytes per update,
BGK collision unless --collision says otherwise) through the same C ABI, so
that the MR/ST speed-up of the paper is measured on B200.

Timing: W untimed warm-up steps; K steps bracketed by barrier +
cuda.synchronize, timed with CUDA events on the stream the kernels are
launched on; max over ranks.  The state (805 MB per buffer) exceeds the
126 MB L2, so no flush is needed between steps.  nvidia-smi clocks are
sampled during the timed region.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time
from pathlib import Path

ROOT = Path(__file__).resolve().parent
sys.path.insert(0, str(ROOT))

import numpy as np  # noqa: E402

from paper_conf_sc_valero_laravgr23_b200 import configs, roofline  # noqa: E402

METRIC = "MLUPS (million lattice-node updates per second, whole job)"
UNIT = "MLUPS"


def load_peaks():
    p = ROOT / "MEASURED_PEAKS.json"
    if p.exists():
        d = json.loads(p.read_text())
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def build_config(name, precision, n_ranks):
    if name == "C5":
        # C5w: one 1024 x 1024 x 128 slab per GPU of the 1024^3 channel
        # (the full 1024^3 fp64 state, 172 GB in two copies, is the P = 8 weak point)
        c = configs.c5(nz=128 * n_ranks)
        c.precision = precision
        return c
    c = configs.ALL[name]() if name != "C2" else configs.c2(precision)
    c.precision = precision
    if n_ranks > 1:
        # weak scaling: one slab of the single-GPU workload per rank along the slab axis
        if c.D == 2:
            c.ny *= n_ranks
        else:
            c.nz *= n_ranks
    return c


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled every 200 ms."""

    FIELDS = ("clocks.sm,clocks.max.sm,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index = index
        self.rows = []
        self.proc = None

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}",
                                          "--format=csv,noheader,nounits", "-lms", "200"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.thread = threading.Thread(target=self._read, daemon=True)
            self.thread.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append([x.strip() for x in line.split(",")])

    def stop(self):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=2)
            except Exception:
                self.proc.kill()
            self.thread.join(timeout=2)
        sm = [float(r[0]) for r in self.rows if len(r) >= 7 and r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in self.rows if len(r) >= 7 and r[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in self.rows if len(r) >= 7 for i in range(4) if r[3 + i] == "Active"})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(sm)}


def cpu_baseline(c, seconds=12.0, max_side=1024):
    """The oracle as it stands on this host's cores, on a bounded sample of
    the workload: the same lattice / regularization / boundary kinds / tau on
    a max_side^D sub-domain, stepped until ~`seconds` of CPU work."""
    import oracle
    threads = oracle.max_threads()
    nx, ny = min(c.nx, max_side), min(c.ny, max_side)
    nz = 1 if c.D == 2 else min(c.nz, max(8, max_side // 8))
    sub = configs.Config(c.name, c.lattice, c.regularization, nx, ny, nz, c.tau, "fp64", c.boundary, c.init, c.U)
    b = {k: dict(v) for k, v in sub.boundary.items()}
    for v in b.values():
        v.pop("u_profile", None)  # profile sized for the full face; sample uses uniform inflow
        if v["kind"] == "velocity":
            v["u"] = [c.U, 0, 0]
    o = oracle.Oracle(c.lattice, nx, ny, nz, c.tau, c.regularization, b, threads=threads)
    o.set_moments(sub.initial_moments())
    o.step(1)  # warm-up
    nodes = nx * ny * (1 if c.D == 2 else nz)
    steps, t0 = 0, time.perf_counter()
    while time.perf_counter() - t0 < seconds:
        o.step(1)
        steps += 1
    dt = time.perf_counter() - t0
    return {"value": nodes * steps / dt / 1e6, "unit": UNIT, "cores": threads, "kind": "oracle",
            "sample": f"{c.lattice}-{c.regularization} {'x'.join(map(str, (nx, ny) if c.D == 2 else (nx, ny, nz)))} "
                      f"sub-domain of {c.name}, {steps} steps in {dt:.1f} s, OpenMP {threads} threads"}


def _oracle_sample(c, side, threads):
    import oracle
    nx, ny = min(c.nx, side), min(c.ny, side)
    nz = 1 if c.D == 2 else min(c.nz, max(8, side // 8))
    sub = configs.Config(c.name, c.lattice, c.regularization, nx, ny, nz, c.tau, "fp64", c.boundary, c.init, c.U)
    b = {k: dict(v) for k, v in sub.boundary.items()}
    for v in b.values():
        v.pop("u_profile", None)  # the sample uses a uniform inflow of the config's U
        if v["kind"] == "velocity":
            v["u"] = [c.U, 0, 0]
    o = oracle.Oracle(c.lattice, nx, ny, nz, c.tau, c.regularization, b, threads=threads)
    o.set_moments(sub.initial_moments())
    return o, (nx, ny, nz), nx * ny * (1 if c.D == 2 else nz)


def run_reference(args, rank, world):
    """--impl reference: the CPU oracle (this tier's reference arm), rank 0 only.
    Each step is one oracle timestep on a sub-domain of the workload sized so
    that the K timed steps take about --ref-seconds on this host."""
    if rank != 0:
        return
    import oracle
    c = build_config(args.config, args.precision, 1)
    threads = oracle.max_threads()
    # probe the host rate on a 256^2 (3D: 64^2 x 8) sample, then size the sample
    o, _, nodes = _oracle_sample(c, 256 if c.D == 2 else 64, threads)
    t0 = time.perf_counter()
    o.step(2)
    rate = 2 * nodes / (time.perf_counter() - t0)  # node updates / s
    budget = rate * args.ref_seconds / max(1, args.steps)
    side = int(budget ** 0.5) if c.D == 2 else int((budget / 8) ** 0.5)
    side = max(16, min(args.ref_side, side))
    o, dims, nodes = _oracle_sample(c, side, threads)
    o.step(args.warmup)
    t0 = time.perf_counter()
    o.step(args.steps)
    dt = time.perf_counter() - t0
    v = nodes * args.steps / dt / 1e6
    sample = (f"{c.lattice}-{c.regularization} {'x'.join(map(str, dims[:c.D]))} sub-domain of {c.name} "
              f"(same faces and tau) per step, {args.steps} steps in {dt:.2f} s, OpenMP {threads} threads")
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": dt / args.steps * 1e3, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": workload_config(c, world),
            "cpu_baseline": {"value": v, "unit": UNIT, "cores": threads, "kind": "oracle", "sample": sample},
            "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def workload_config(c, world):
    dims = f"{c.nx}x{c.ny}" if c.D == 2 else f"{c.nx}x{c.ny}x{c.nz}"
    coll = "BGK" if c.regularization == "bgk" else f"{c.regularization}-regularized"
    return {"workload": f"{c.name}: {c.lattice} {coll} "
                        f"{'lid-driven cavity' if 'y+' in c.boundary and c.boundary['y+']['kind'] == 'moving_wall' else ('channel' if c.name == 'C5' else 'flow')} "
                        f"{dims} {c.precision}",
            "lattice": c.lattice, "regularization": c.regularization, "grid": dims, "tau": c.tau,
            "precision": c.precision, "nodes": c.nodes,
            "parallelism": f"{'y' if c.D == 2 else 'z'}-slab x{world}" if world > 1 else "1 GPU",
            "l2": "state larger than the 126 MB L2 (no flush needed)" if c.nodes * 2 * roofline.M_OF[c.lattice]
                  * roofline.WORD[c.precision] > 126e6 else "state fits in L2"}


def traffic_from_profiles(c, method="MR"):
    """dram bytes per launch of the fused kernel from the committed ncu summary."""
    p = ROOT / "profiles" / "ncu_summary.json"
    if not p.exists():
        return None
    try:
        d = json.loads(p.read_text())
        key = f"{c.name}-{c.lattice}-{c.regularization}-{c.precision}-{c.nx}x{c.ny}x{c.nz if c.D == 3 else 1}"
        if method != "MR":
            key = f"{method}-{key}"
        return d.get(key, {}).get("dram_bytes_per_launch")
    except Exception:
        return None


def run_gpu(args, rank, world, local_rank):
    import torch
    from paper_conf_sc_valero_laravgr23_b200 import mrlbm

    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    dist = None
    if world > 1:
        import torch.distributed as dist
        dist.init_process_group("nccl", device_id=dev)
    c = build_config(args.config, args.precision, world)
    st = args.method == "ST"
    if st:
        if world > 1:
            raise SystemExit("--method ST runs on one GPU (the distribution representation is single-rank)")
        # the paper's ST reference collides with BGK (Alg. 1); --collision overrides
        c.regularization = args.collision or "bgk"
        for v in c.boundary.values():
            if v["kind"] in ("velocity", "pressure"):
                raise SystemExit("--method ST: open faces are not implemented for the distribution representation")
    elif args.collision:
        c.regularization = args.collision
    nccl_id = None
    p2p = world > 1 and args.transport == "p2p"
    if world > 1 and not p2p:
        idt = torch.zeros(128, dtype=torch.uint8, device=dev)
        if rank == 0:
            idt.copy_(torch.frombuffer(bytearray(mrlbm.nccl_unique_id()), dtype=torch.uint8).to(dev))
        dist.broadcast(idt, 0)
        nccl_id = bytes(idt.cpu().numpy().tobytes())
    stream = torch.cuda.Stream(device=dev)
    s = mrlbm.Solver(c.lattice, c.nx, c.ny, c.nz, c.tau, c.regularization, c.boundary, precision=c.precision,
                     device=local_rank, stream=stream.cuda_stream, rank=rank, nranks=world, nccl_id=nccl_id,
                     representation="distributions" if st else "moments", transport="p2p" if p2p else "nccl")
    if p2p:
        # halo pushes through peer memory (CUDA IPC over NVLink): exchange the handles once
        from paper_conf_sc_valero_laravgr23_b200 import distributed as sd
        handles = [None] * world
        dist.all_gather_object(handles, s.p2p_handle())
        sd.p2p_connect(s, handles, sd.slab_axis_periodic(c.boundary, c.D))
    # initial state: this rank's slab of the seeded initial moments
    m0 = c.initial_moments()
    sl = slice(s.offset, s.offset + s.n_local)
    m_local = np.ascontiguousarray(m0[:, sl] if c.D == 2 else m0[:, sl])
    del m0
    s.set_moments(m_local)
    nodes_local = s.N

    def barrier():
        if dist is not None:
            dist.barrier()

    # warm-up (also captures the step graphs)
    s.step(args.warmup)
    s.sync()
    barrier()
    torch.cuda.synchronize(dev)
    clk = ClockSampler(local_rank)
    clk.start()
    # keep the GPU busy (untimed steps, the same count on every rank) for
    # ~0.5 s while the sampler starts: idling here let the clocks/power state
    # drop, and a short timed region then paid the ramp (measured: K=1000 C2
    # read 43-53k MLUPS while e2e, timed later, read 53k)
    t_hot = time.perf_counter()
    s.step(32)
    s.sync()
    chunks = torch.tensor([max(1.0, 0.5 / max(time.perf_counter() - t_hot, 1e-4))], device=dev, dtype=torch.float64)
    if dist is not None:
        dist.all_reduce(chunks, op=dist.ReduceOp.MAX)
    for _ in range(min(int(chunks.item()), 4096)):
        s.step(32)
    s.sync()
    barrier()
    k0 = s.launch_count()
    with torch.cuda.stream(stream):
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        barrier()
        torch.cuda.synchronize(dev)
        e0.record(stream)
        s.step(args.steps)
        e1.record(stream)
        e1.synchronize()
        torch.cuda.synchronize(dev)
        barrier()
    ms = e0.elapsed_time(e1)
    clocks = clk.stop()
    launches = s.launch_count() - k0
    if dist is not None:
        t = torch.tensor([ms], device=dev, dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
    total_nodes = nodes_local * world
    value = total_nodes * args.steps / (ms * 1e-3) / 1e6
    ms_step = ms / args.steps

    # end to end through the public C-ABI with host buffers: upload (pinned),
    # K steps, download -- all inside the timed region
    pinned_in = torch.from_numpy(m_local).pin_memory()
    pinned_out = torch.empty_like(pinned_in).pin_memory()
    import ctypes
    dp = ctypes.POINTER(ctypes.c_double)
    barrier()
    torch.cuda.synchronize(dev)
    t0 = time.perf_counter()
    mrlbm._check(mrlbm.lib.mrlbm_set_moments(s._h, ctypes.cast(pinned_in.data_ptr(), dp), pinned_in.numel()), "set")
    s.step(args.steps)
    mrlbm._check(mrlbm.lib.mrlbm_get_moments(s._h, ctypes.cast(pinned_out.data_ptr(), dp), pinned_out.numel()), "get")
    barrier()
    te = time.perf_counter() - t0
    if dist is not None:
        t = torch.tensor([te], device=dev, dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        te = float(t.item())
    e2e = {"value": total_nodes * args.steps / te / 1e6, "unit": UNIT,
           "h2d_bytes_per_step": pinned_in.numel() * 8 * world / args.steps,
           "d2h_bytes_per_step": pinned_out.numel() * 8 * world / args.steps,
           "job": "mrlbm_set_moments (pinned host) + mrlbm_step(K) + mrlbm_get_moments (pinned host)"}
    finite_ok = True
    try:
        s.check_finite()
    except Exception:
        finite_ok = False

    # roofline of the dominant (fused step) kernel: algorithmic bytes 2 M w per node
    peak, peak_src = load_peaks()
    bpl = roofline.bytes_per_lup(c.lattice, "ST" if st else "MR", c.precision)
    launches_per_step = max(1, round(launches / args.steps))
    achieved = nodes_local * bpl / (ms_step * 1e-3) / 1e9
    tr = traffic_from_profiles(c, args.method)
    line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "f64" if c.precision == "fp64" else "f32", "data": "synthetic",
            "config": dict(workload_config(c, world), method=args.method,
                           **({"transport": args.transport} if world > 1 else {})),
            "per_gpu_mlups": value / world,
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
                         "traffic": tr, "peak_source": peak_src,
                         "algorithmic_bytes_per_lup": bpl, "lups_per_launch": nodes_local,
                         "roofline_mlups_per_gpu": peak * 1e9 / bpl / 1e6,
                         "note": f"achieved = {bpl} B/LUP x {nodes_local} LUP / mean step time "
                                 f"({launches_per_step} fused launch(es) per step)"},
            "clocks": clocks, "e2e": e2e, "gpu_launches": launches, "kernel": s.kernel_config(),
            "finite": finite_ok}
    if rank == 0 and not args.no_cpu_baseline:
        line["cpu_baseline"] = cpu_baseline(c, seconds=args.cpu_seconds)
    s.close()
    if rank == 0:
        print(json.dumps(line), flush=True)
    if dist is not None:
        dist.barrier()
        dist.destroy_process_group()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=4000)
    ap.add_argument("--warmup", type=int, default=64)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="C2", choices=list(configs.ALL))
    ap.add_argument("--precision", default="fp64", choices=["fp64", "fp32"])
    ap.add_argument("--method", default="MR", choices=["MR", "ST"],
                    help="MR = the paper's moment representation (default); ST = its distribution baseline")
    ap.add_argument("--collision", default=None, choices=["projective", "recursive", "bgk"],
                    help="override the collision (ST default: bgk, the paper's Alg. 1)")
    ap.add_argument("--transport", default="nccl", choices=["nccl", "p2p"],
                    help="N > 1 halo transport: NCCL send/recv (default) or peer-memory pushes fused into the step")
    ap.add_argument("--cpu-seconds", type=float, default=12.0)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--ref-side", type=int, default=1024, help="reference arm: max sample sub-domain side")
    ap.add_argument("--ref-seconds", type=float, default=60.0, help="reference arm: target timed seconds")
    args = ap.parse_args()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if args.warmup < 3:
        args.warmup = 3
    if args.impl == "reference":
        run_reference(args, rank, world)
    else:
        run_gpu(args, rank, world, local_rank)


if __name__ == "__main__":
    main()
