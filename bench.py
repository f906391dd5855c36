"""bench.py -- MR-LBM throughput on B200 (BASELINE.json metric: MLUPS per GPU
and whole box; achieved HBM GB/s vs peak).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config C2|C3|C4|C5|C1] [--precision fp64|fp32]
  python bench.py --gpus 8 [--strong]        # spawns 8 ranks itself when not under torchrun
  python bench.py --impl reference ...      # the CPU oracle arm (bounded sample)
  python bench.py --method ST [--collision bgk] ...  # the paper's ST baseline on the GPU

A "step" is one timestep of the whole hot path (load moments -> collide ->
reconstruct -> stream -> boundaries -> moments -> store, plus the slab halo
exchange at N > 1) over the whole domain.

Workloads (BASELINE.json configs):
  N = 1 default   C2: D2Q9 recursive-regularized lid-driven cavity 4096^2, fp64
                  (configs[1], the config the metric is quoted on)
  N > 1 default   C5 weak scaling: D3Q19 recursive channel, one 1024 x 1024 x 128
                  z-slab per GPU (N = 8: the 1024^3 channel), NCCL halo exchange
  --strong        the config's global size split over the N ranks (C5: 1024^3,
                  C4: 512^3 at 2 GPUs)
The N = 1 line also carries the C1 record (D2Q9 Poiseuille 128 x 64, 1000 steps:
GPU and oracle wall seconds, parity) -- configs[0].

Timing: W untimed warm-up steps, ~0.5 s of untimed busy steps (clock ramp),
then R >= 5 repetitions of EXACTLY K steps, each bracketed by barrier +
cuda.synchronize on both sides and timed with CUDA events on the stream the
kernels run on; per repetition the max over ranks; `value` = the median
repetition.  A second record times 5 blocks of >= 200 ms each (`sustained`).
Every state exceeds the 126 MB L2 except C1, so no flush is needed between
steps (`config.l2`).  nvidia-smi clocks are sampled during the timed region.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import socket
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
SPEC_HBM_GBS = 8000.0  # B200 spec (DGX figure)
SMS = 148


def load_peaks():
    p = ROOT / "MEASURED_PEAKS.json"
    if p.exists():
        d = json.loads(p.read_text())
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def default_precision(name):
    return "fp32" if name == "C4" else "fp64"


def build_config(name, precision, n_ranks, strong=False):
    """The workload of one bench line.  Weak scaling (default): each rank owns
    one copy of the single-GPU slab along the slab axis; strong: the config's
    global size is split."""
    if name == "C5":
        # C5w: one 1024 x 1024 x 128 slab per GPU of the channel;
        # --strong: the 1024^3 channel split over the ranks
        c = configs.c5(nz=1024 if strong else 128 * n_ranks)
    elif name == "C2":
        c = configs.c2(precision)
    else:
        c = configs.ALL[name]()
    c.precision = precision
    if n_ranks > 1 and not strong and name != "C5":
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


# ---------------------------------------------------------------- CPU (oracle) legs
def host_cores():
    return len(os.sched_getaffinity(0))


def cpu_model():
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for line in out.splitlines():
            if line.startswith("Model name:"):
                return line.split(":", 1)[1].strip()
    except Exception:
        pass
    try:
        for line in Path("/proc/cpuinfo").read_text().splitlines():
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except Exception:
        pass
    return "unknown"


def _oracle_sample(c, side, threads):
    import oracle
    nx, ny = min(c.nx, side), min(c.ny, side)
    nz = 1 if c.D == 2 else min(c.nz, max(8, side // 8))
    if c.init == "taylor_green_3d":  # the Taylor-Green field is defined on a cube
        nx = ny = nz = min(c.nx, max(16, side // 2))
    sub = configs.Config(c.name, c.lattice, c.regularization, nx, ny, nz, c.tau, "fp64", c.boundary, c.init, c.U)
    b = {k: dict(v) for k, v in sub.boundary.items()}
    for v in b.values():
        v.pop("u_profile", None)  # the sample uses a uniform inflow of the config's U
        if v["kind"] == "velocity":
            v["u"] = [c.U, 0, 0]
    o = oracle.Oracle(c.lattice, nx, ny, nz, c.tau, c.regularization, b, threads=threads)
    o.set_moments(sub.initial_moments())
    return o, (nx, ny, nz), nx * ny * (1 if c.D == 2 else nz)


def _oracle_leg(c, seconds, threads, side):
    o, dims, nodes = _oracle_sample(c, side, threads)
    o.step(1)  # warm-up
    steps, t0 = 0, time.perf_counter()
    while time.perf_counter() - t0 < seconds:
        o.step(1)
        steps += 1
    dt = time.perf_counter() - t0
    return nodes * steps / dt / 1e6, steps, dt, dims


def cpu_baseline(c, seconds=16.0):
    """The oracle as it stands on this host's cores, on a bounded sample of the
    workload (same lattice / regularization / boundary kinds / tau on a
    sub-domain), two legs: all cores of the affinity mask, and one thread."""
    cores = host_cores()
    side = 1024 if c.D == 2 else 128
    v_all, st_all, dt_all, dims = _oracle_leg(c, seconds / 2, cores, side)
    v_one, st_one, dt_one, dims1 = _oracle_leg(c, seconds / 2, 1, 256 if c.D == 2 else 48)
    shape = lambda d: "x".join(map(str, d[:c.D]))  # noqa: E731
    return {"value": v_all, "unit": UNIT, "cores": cores, "kind": "oracle", "cpu_model": cpu_model(),
            "sample": f"{c.lattice}-{c.regularization} {shape(dims)} sub-domain of {c.name} (same faces, tau), "
                      f"{st_all} steps in {dt_all:.1f} s on {cores} threads (OpenMP over nodes)",
            "single_thread": {"value": v_one, "unit": UNIT, "cores": 1,
                              "sample": f"{shape(dims1)} sub-domain, {st_one} steps in {dt_one:.1f} s"}}


def c1_record(local_rank):
    """BASELINE configs[0] (C1): D2Q9 projective Poiseuille 128 x 64, fp64, 1000
    steps -- wall seconds of the GPU (through the C ABI, host buffers) and of
    the oracle on all host cores, and their parity (SURVEY 8(c) metric)."""
    import oracle
    from paper_conf_sc_valero_laravgr23_b200 import mrlbm
    c = configs.c1()
    m0 = c.initial_moments()
    with mrlbm.Solver(c.lattice, c.nx, c.ny, 1, c.tau, c.regularization, c.boundary, device=local_rank) as s:
        s.set_moments(m0)
        s.step(64)   # warm-up (captures the step graphs)
        s.sync()
        t0 = time.perf_counter()
        s.set_moments(m0)
        s.step(c.steps)
        got = s.get_moments()
        t_gpu = time.perf_counter() - t0
    cores = host_cores()
    o = oracle.Oracle(c.lattice, c.nx, c.ny, 1, c.tau, c.regularization, c.boundary, threads=cores)
    t0 = time.perf_counter()
    o.set_moments(m0)
    o.step(c.steps)
    ref = o.get_moments()
    t_cpu = time.perf_counter() - t0
    err = {g: float(np.abs(got[i] - ref[i]).max() / np.abs(ref[i]).max())
           for g, i in (("rho", [0]), ("u", [1, 2]), ("Pi", [3, 4, 5]))}
    return {"workload": "C1: D2Q9 projective-regularized Poiseuille channel 128x64 fp64, 1000 steps",
            "gpu_seconds": t_gpu, "oracle_seconds": t_cpu, "oracle_cores": cores,
            "gpu_job": "mrlbm_set_moments + mrlbm_step(1000) + mrlbm_get_moments (host buffers), wall clock",
            "parity_group_errors": err, "parity_ok": max(err.values()) <= 1e-11}


# ---------------------------------------------------------------- reference arm
def run_reference(args, rank, world):
    """--impl reference: the CPU oracle (this tier's reference arm), rank 0 only.
    Each step is one oracle timestep on a sub-domain of the workload sized so
    that the K timed steps take about --ref-seconds on this host."""
    if rank != 0:
        return
    name = args.config or ("C2" if world == 1 else "C5")
    c = build_config(name, args.precision or default_precision(name), 1)
    threads = host_cores()
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
            "scaling": "strong" if args.strong else "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": workload_config(c, world, args.strong),
            "cpu_baseline": {"value": v, "unit": UNIT, "cores": threads, "kind": "oracle", "sample": sample,
                             "cpu_model": cpu_model()},
            "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def workload_config(c, world, strong=False):
    dims = f"{c.nx}x{c.ny}" if c.D == 2 else f"{c.nx}x{c.ny}x{c.nz}"
    coll = "BGK" if c.regularization == "bgk" else f"{c.regularization}-regularized"
    kind = ("lid-driven cavity" if "y+" in c.boundary and c.boundary["y+"]["kind"] == "moving_wall"
            else ("channel" if c.name in ("C5", "C1") else ("Taylor-Green vortex" if c.name == "C3" else "flow")))
    state_bytes = c.nodes * 2 * roofline.M_OF[c.lattice] * roofline.WORD[c.precision]
    return {"workload": f"{c.name}: {c.lattice} {coll} {kind} {dims} {c.precision}",
            "lattice": c.lattice, "regularization": c.regularization, "grid": dims, "tau": c.tau,
            "precision": c.precision, "nodes": c.nodes,
            "parallelism": (f"{'y' if c.D == 2 else 'z'}-slab x{world} ({'strong' if strong else 'weak'})"
                            if world > 1 else "1 GPU"),
            "l2": ("state larger than the 126 MB L2 (no flush needed)" if state_bytes / max(world, 1) > 126e6
                   else "state fits in L2")}


def alu_from_profiles(c, method, nodes_local):
    """Issue / FP64 / FMA-pipe ceilings of the fused kernel from the committed ncu
    summary: the MLUPS at which that unit would be 100% busy with the kernel's
    own instruction mix (ncu: unit-active fraction x duration per launch)."""
    p = ROOT / "profiles" / "ncu_summary.json"
    if not p.exists():
        return None, None
    try:
        d = json.loads(p.read_text())
        key = f"{c.name}-{c.lattice}-{c.regularization}-{c.precision}-{c.nx}x{c.ny}x{c.nz if c.D == 3 else 1}"
        if method != "MR":
            key = f"{method}-{key}"
        e = d.get(key)
        if not e:
            return None, None
        dur = e["duration"]
        lups = nodes_local
        out = {"source": f"profiles/ncu_summary.json[{key}] ({e.get('tag', '')})"}
        for name, k in (("issue", "issue_active_pct"), ("fp64_pipe", "fp64_pipe_pct"), ("fma_pipe", "fma_pipe_pct")):
            if e.get(k):
                out[f"{name}_ceiling_mlups"] = lups / (dur * e[k] / 100.0) / 1e6
        if e.get("warp_inst"):
            out["warp_inst_per_lup"] = e["warp_inst"] / lups
        ceil = [v for k, v in out.items() if k.endswith("_ceiling_mlups")]
        if ceil:
            out["alu_ceiling_mlups"] = min(ceil)
        return out, e.get("dram_bytes_per_launch")
    except Exception:
        return None, None


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


# ---------------------------------------------------------------- GPU arm
def run_gpu(args, rank, world, local_rank):
    import torch
    from paper_conf_sc_valero_laravgr23_b200 import mrlbm

    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    dist = None
    if world > 1:
        import torch.distributed as dist
        dist.init_process_group("nccl", device_id=dev)
    name = args.config or ("C2" if world == 1 else "C5")
    c = build_config(name, args.precision or default_precision(name), world, args.strong)
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
    comm = s.comm_info()
    if p2p:
        # halo pushes through peer memory (CUDA IPC over NVLink): exchange the handles once
        from paper_conf_sc_valero_laravgr23_b200 import distributed as sd
        handles = [None] * world
        dist.all_gather_object(handles, s.p2p_handle())
        sd.p2p_connect(s, handles, sd.slab_axis_periodic(c.boundary, c.D))
    # initial state: this rank's slab of the seeded initial moments (generated slab-only)
    m_local = np.ascontiguousarray(c.initial_moments(lo=s.offset, hi=s.offset + s.n_local))
    s.set_moments(m_local)
    nodes_local = s.N

    def barrier():
        if dist is not None:
            dist.barrier()

    def max_over_ranks(x):
        if dist is None:
            return x
        t = torch.tensor([x], device=dev, dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    # warm-up (also captures the step graphs)
    s.step(args.warmup)
    s.sync()
    barrier()
    torch.cuda.synchronize(dev)
    clk = ClockSampler(local_rank)
    clk.start()
    # keep the GPU busy (untimed steps, the same count on every rank) for
    # ~0.5 s while the sampler starts: an idle GPU drops its clocks and a short
    # timed region then pays the ramp (round 1: K=1000 C2 read 43-53k MLUPS)
    t_hot = time.perf_counter()
    s.step(32)
    s.sync()
    chunks = max_over_ranks(max(1.0, 0.5 / max(time.perf_counter() - t_hot, 1e-4)))
    for _ in range(min(int(chunks), 4096)):
        s.step(32)
    s.sync()
    barrier()

    def timed(nsteps):
        """one timed region of exactly nsteps steps: barrier + sync on both sides,
        CUDA events on the kernels' stream; max over ranks (ms)"""
        with torch.cuda.stream(stream):
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            barrier()
            torch.cuda.synchronize(dev)
            e0.record(stream)
            s.step(nsteps)
            e1.record(stream)
            e1.synchronize()
            torch.cuda.synchronize(dev)
            barrier()
        return max_over_ranks(e0.elapsed_time(e1))

    reps = max(5, args.reps)
    k0 = s.launch_count()
    rep_ms = [timed(args.steps) for _ in range(reps)]
    launches = (s.launch_count() - k0) // reps
    s.sync()
    ms = statistics.median(rep_ms)
    ms_step = ms / args.steps
    # sustained: 5 blocks of >= 200 ms each
    blk_steps = max(32, int(math.ceil(200.0 / max(ms_step, 1e-6) / 32.0)) * 32)
    blk_ms = [timed(blk_steps) for _ in range(5)]
    s.sync()
    clocks = clk.stop()
    total_nodes = c.nodes  # every rank's slab (weak: world x the per-GPU slab)
    value = total_nodes * args.steps / (ms * 1e-3) / 1e6
    blk_mlups = [total_nodes * blk_steps / (t * 1e-3) / 1e6 for t in blk_ms]

    # end to end through the public C-ABI with host buffers: upload (pinned),
    # K steps, download -- all inside the timed region
    if args.no_e2e:  # side runs whose host state would not fit twice in pinned memory
        return finish_line(args, s, c, st, world, rank, local_rank, dist, name, nodes_local, rep_ms, ms_step, ms,
                           launches, blk_steps, blk_ms, blk_mlups, clocks, value, comm, None)
    import torch as _t
    pinned_in = _t.from_numpy(m_local).pin_memory()
    pinned_out = _t.empty_like(pinned_in).pin_memory()
    del m_local
    import ctypes
    dp = ctypes.POINTER(ctypes.c_double)
    barrier()
    torch.cuda.synchronize(dev)
    t0 = time.perf_counter()
    mrlbm._check(mrlbm.lib.mrlbm_set_moments(s._h, ctypes.cast(pinned_in.data_ptr(), dp), pinned_in.numel()), "set")
    s.step(args.steps)
    mrlbm._check(mrlbm.lib.mrlbm_get_moments(s._h, ctypes.cast(pinned_out.data_ptr(), dp), pinned_out.numel()), "get")
    barrier()
    te = max_over_ranks(time.perf_counter() - t0)
    s.sync()
    e2e = {"value": total_nodes * args.steps / te / 1e6, "unit": UNIT,
           "h2d_bytes_per_step": roofline.M_OF[c.lattice] * 8 * c.nodes / args.steps,
           "d2h_bytes_per_step": roofline.M_OF[c.lattice] * 8 * c.nodes / args.steps,
           "job": "mrlbm_set_moments (pinned host) + mrlbm_step(K) + mrlbm_get_moments (pinned host), wall clock"}
    return finish_line(args, s, c, st, world, rank, local_rank, dist, name, nodes_local, rep_ms, ms_step, ms,
                       launches, blk_steps, blk_ms, blk_mlups, clocks, value, comm, e2e)


def finish_line(args, s, c, st, world, rank, local_rank, dist, name, nodes_local, rep_ms, ms_step, ms, launches,
                blk_steps, blk_ms, blk_mlups, clocks, value, comm, e2e):
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
    alu, traffic = alu_from_profiles(c, args.method, nodes_local)
    hbm_ceiling = peak * 1e9 / bpl / 1e6
    rl = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
          "traffic": traffic, "peak_source": peak_src, "frac_of_spec": achieved / SPEC_HBM_GBS,
          "spec_gbs": SPEC_HBM_GBS, "algorithmic_bytes_per_lup": bpl, "lups_per_launch": nodes_local,
          "roofline_mlups_per_gpu": hbm_ceiling,
          "note": f"achieved = {bpl} B/LUP x {nodes_local} LUP / median step time "
                  f"({launches_per_step} launch(es) per step on this rank)"}
    if alu:
        rl["alu"] = alu
        if alu.get("alu_ceiling_mlups") and alu["alu_ceiling_mlups"] < hbm_ceiling:
            rl["co_bound"] = (f"ALU ceiling {alu['alu_ceiling_mlups']:.0f} MLUPS < HBM ceiling "
                              f"{hbm_ceiling:.0f} MLUPS: issue/FP-pipe bound at this instruction mix")
    line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": True,
            "scaling": "strong" if args.strong else "weak",
            "vs_baseline": None, "dtype": "f64" if c.precision == "fp64" else "f32", "data": "synthetic",
            "config": dict(workload_config(c, world, args.strong), method=args.method,
                           **({"transport": args.transport} if world > 1 else {})),
            "per_gpu_mlups": value / world,
            "reps": {"n": len(rep_ms), "steps_each": args.steps, "ms_per_step": [t / args.steps for t in rep_ms],
                     "median_ms_per_step": ms_step,
                     "spread_pct": 100.0 * (max(rep_ms) - min(rep_ms)) / ms},
            "sustained": {"blocks": 5, "steps_per_block": blk_steps, "block_ms": blk_ms,
                          "mlups": blk_mlups, "median_mlups": statistics.median(blk_mlups)},
            "roofline": rl, "clocks": clocks, "gpu_launches": launches,
            "kernel": s.kernel_config(), "finite": finite_ok,
            "gpus_active": world, "comm": comm}
    if e2e is not None:
        line["e2e"] = e2e
    else:
        line["e2e_skipped"] = "--no-e2e (side run: the host state does not fit twice in pinned memory)"
    s.close()
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        try:
            line["cpu_baseline"] = cpu_baseline(c, seconds=args.cpu_seconds)
        except Exception as e:  # the GPU line stands without it
            line["cpu_baseline"] = {"error": repr(e)[:300]}
        if name == "C2" and not st:
            line["c1"] = c1_record(local_rank)
    if world != args.gpus:
        raise SystemExit(f"bench.py: ran on {world} rank(s) but --gpus {args.gpus}: no line printed")
    if rank == 0:
        print(json.dumps(line), flush=True)
    if dist is not None:
        dist.barrier()
        dist.destroy_process_group()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=1000)
    ap.add_argument("--warmup", type=int, default=64)
    ap.add_argument("--reps", type=int, default=5, help="timed repetitions of K steps (>= 5; median reported)")
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default=None, choices=list(configs.ALL),
                    help="default: C2 at N = 1, C5 (weak, 1024 x 1024 x 128 per GPU) at N > 1")
    ap.add_argument("--strong", action="store_true", help="split the config's global size over the N ranks")
    ap.add_argument("--precision", default=None, choices=["fp64", "fp32"], help="default: the config's")
    ap.add_argument("--method", default="MR", choices=["MR", "ST"],
                    help="MR = the paper's moment representation (default); ST = its distribution baseline")
    ap.add_argument("--collision", default=None, choices=["projective", "recursive", "bgk"],
                    help="override the collision (ST default: bgk, the paper's Alg. 1)")
    ap.add_argument("--transport", default="nccl", choices=["nccl", "p2p"],
                    help="N > 1 halo transport: NCCL send/recv (default) or peer-memory pushes fused into the step")
    ap.add_argument("--cpu-seconds", type=float, default=16.0)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true", help="skip the host-buffer e2e leg (side runs only)")
    ap.add_argument("--ref-side", type=int, default=1024, help="reference arm: max sample sub-domain side")
    ap.add_argument("--ref-seconds", type=float, default=60.0, help="reference arm: target timed seconds")
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3
    if "WORLD_SIZE" not in os.environ and args.gpus > 1:
        # not under torchrun: start one rank per GPU ourselves (same arguments)
        cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
               "--master-addr", "127.0.0.1", "--master-port", str(_free_port()), str(Path(__file__).resolve()),
               *sys.argv[1:]]
        sys.exit(subprocess.call(cmd))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        run_reference(args, rank, world)
        return
    if world != args.gpus:
        sys.stderr.write(f"bench.py: WORLD_SIZE={world} but --gpus {args.gpus}; refusing to print a line\n")
        sys.exit(2)
    run_gpu(args, rank, world, local_rank)


if __name__ == "__main__":
    main()
