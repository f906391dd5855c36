"""Summarise ncu reports of the fused step kernel into profiles/ (JSON + markdown).

  python tools/ncu_summary.py KEY gpurun_out/prof_C2.ncu-rep [KEY2 rep2 ...] --tag r01 [--bench bench.jsonl]

KEY is the bench's workload key (e.g. C2-D2Q9-recursive-fp64-4096x4096x1);
the JSON (profiles/ncu_summary.json) is what bench.py reads for
roofline.traffic (dram bytes per launch).
"""
import csv
import io
import json
import subprocess
import sys
from pathlib import Path

ROOT = Path(__file__).resolve().parents[1]
METRICS = {
    "gpu__time_duration.sum": "duration",
    "dram__bytes_read.sum": "dram_read",
    "dram__bytes_write.sum": "dram_write",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed": "dram_pct_peak",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed": "sm_pct_peak",
    "launch__registers_per_thread": "registers",
    "launch__block_size": "block",
    "launch__grid_size": "grid",
    "sm__warps_active.avg.pct_of_peak_sustained_active": "warps_active_pct",
    "launch__occupancy_limit_registers": "occ_limit_regs",
    "launch__occupancy_limit_shared_mem": "occ_limit_smem",
    "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active": "fp64_pipe_pct",
    "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active": "fma_pipe_pct",
    "smsp__issue_active.avg.pct_of_peak_sustained_active": "issue_active_pct",
    "smsp__inst_executed.sum": "warp_inst",
    "lts__t_sector_hit_rate.pct": "l2_hit_pct",
    "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum": "smem_bank_conflicts",
    "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active": "tensor_pipe_pct",
}
UNIT_SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12,
              "nsecond": 1e-9, "usecond": 1e-6, "msecond": 1e-3, "second": 1,
              "ns": 1e-9, "us": 1e-6, "ms": 1e-3, "s": 1}


def read_rep(path):
    """an .ncu-rep, or the `--page raw --csv` export of one (tools/ncu_capture.sh)"""
    if str(path).endswith(".csv"):
        out = Path(path).read_text()
    else:
        out = subprocess.run(["ncu", "-i", str(path), "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units, vals = rows[0], rows[1], rows[2]
    res = {"kernel": vals[hdr.index("Kernel Name")] if "Kernel Name" in hdr else ""}
    for m, k in METRICS.items():
        if m in hdr:
            i = hdr.index(m)
            v = vals[i].replace(",", "")
            try:
                x = float(v) * UNIT_SCALE.get(units[i], 1)
            except ValueError:
                continue
            res[k] = x
    if "dram_read" in res and "dram_write" in res:
        res["dram_bytes_per_launch"] = res["dram_read"] + res["dram_write"]
        if res.get("duration"):
            res["dram_gbs"] = res["dram_bytes_per_launch"] / res["duration"] / 1e9
    return res


def main():
    args = sys.argv[1:]
    tag = "r01"
    if "--tag" in args:
        i = args.index("--tag")
        tag = args[i + 1]
        del args[i:i + 2]
    summ_path = ROOT / "profiles" / "ncu_summary.json"
    summ = json.loads(summ_path.read_text()) if summ_path.exists() else {}
    md = [f"# ncu --set full summaries ({tag})\n",
          "One launch of the fused step kernel per workload (`ncu --set full --clock-control none "
          "--import-source on -k regex:mrlbm_step -s 5 -c 1`), cold-cache and serialised by ncu.\n",
          "| workload | kernel | time | DRAM bytes/launch | traffic / algorithmic (2 M w per LUP) | DRAM GB/s | "
          "regs | block x grid | warps active % | issue % | fp64 pipe % | fma pipe % | L2 hit % | warp-inst / LUP | "
          "ALU ceiling (MLUPS, unit) |",
          "|---|---|---|---|---|---|---|---|---|---|---|---|---|---|---|"]
    for key, rep in zip(args[0::2], args[1::2]):
        r = read_rep(rep)
        r["tag"] = tag
        r["report"] = Path(rep).name
        summ[key] = r
        # LUPs per launch and algorithmic bytes from the key: C?-LAT-REG-PREC-NXxNYxNZ
        parts = key.split("-")
        lat, prec = parts[1], parts[3]
        nx, ny, nz = (int(v) for v in parts[4].split("x"))
        lups = nx * ny * nz
        M = 6 if lat == "D2Q9" else 10
        alg = 2 * M * (8 if prec == "fp64" else 4) * lups
        r["lups_per_launch"] = lups
        r["algorithmic_bytes_per_launch"] = alg
        dur = r.get("duration", 0) or 1e-30
        ceil = {u: lups / (dur * r[k] / 100.0) / 1e6 for u, k in
                (("issue", "issue_active_pct"), ("fp64", "fp64_pipe_pct"), ("fma", "fma_pipe_pct")) if r.get(k)}
        cu = min(ceil, key=ceil.get) if ceil else None
        md.append(f"| {key} | `{r['kernel'][:60]}` | {r.get('duration', 0) * 1e6:.1f} us | "
                  f"{r.get('dram_bytes_per_launch', 0) / 1e9:.3f} GB | "
                  f"{r.get('dram_bytes_per_launch', 0) / alg:.3f} | {r.get('dram_gbs', 0):.0f} | "
                  f"{r.get('registers', 0):.0f} | {r.get('block', 0):.0f} x "
                  f"{r.get('grid', 0):.0f} | {r.get('warps_active_pct', 0):.1f} | {r.get('issue_active_pct', 0):.1f} | "
                  f"{r.get('fp64_pipe_pct', 0):.1f} | {r.get('fma_pipe_pct', 0):.1f} | {r.get('l2_hit_pct', 0):.1f} | "
                  f"{r.get('warp_inst', 0) / lups:.2f} | "
                  f"{(f'{ceil[cu]:.0f} ({cu})') if cu else '-'} |")
    summ_path.write_text(json.dumps(summ, indent=1, sort_keys=True))
    (ROOT / "profiles" / f"ncu_{tag}.md").write_text("\n".join(md) + "\n")
    print("\n".join(md))


if __name__ == "__main__":
    main()
