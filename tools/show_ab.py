"""one line per bench JSON line of an A/B run (lib tag, workload, MLUPS, roofline fraction, clocks)"""
import json
import sys

for f in sys.argv[1:]:
    for l in open(f):
        try:
            d = json.loads(l)
        except Exception:
            continue
        r = d["roofline"]
        print(f'{d.get("lib", "-"):8s} {d["config"]["workload"][:60]:60s} {d["value"]:8.0f} MLUPS frac {r["frac"]:.3f} '
              f'clk {d["clocks"]["sm_mhz"]} {d["clocks"]["reasons"]} spread {d["reps"]["spread_pct"]:.1f}% '
              f'grid {d["kernel"]["grid_x"]}x{d["kernel"]["grid_y"]}')
