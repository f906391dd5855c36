import json, sys
for f in sys.argv[1:]:
    for l in open(f):
        try:
            d = json.loads(l)
        except Exception:
            continue
        r = d.get("roofline", {})
        k = d.get("kernel", {})
        print(f"{d['config'].get('method','MR'):2s} {d['config']['workload'][:70]:70s} {d['value']:9.0f} MLUPS {d['ms_per_step']:8.3f} ms "
              f"{(r.get('achieved') or 0):7.0f} GB/s frac {(r.get('frac') or 0):.3f} clk {d.get('clocks', {}).get('sm_mhz')} "
              f"{d.get('clocks', {}).get('reasons')} e2e {d.get('e2e', {}).get('value', 0):.0f} grid {k.get('grid_x')}x{k.get('grid_y')}")
