"""Summarise an ncu launch list (--metrics gpu__time_duration.sum --csv) into markdown.

  python tools/launch_summary.py gpurun_out/launches_TAG_C2.csv "title" > profiles/launches_TAG_C2.md
"""
import collections
import csv
import sys

rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 10]
h = rows[0]
ik, iv, iu = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
scale = {"ns": 1e-3, "us": 1.0, "usecond": 1.0, "nsecond": 1e-3, "ms": 1e3, "msecond": 1e3}
tot = collections.Counter()
cnt = collections.Counter()
for r in rows[1:]:
    k = r[ik][:60]
    tot[k] += float(r[iv].replace(",", "")) * scale.get(r[iu], 1.0)
    cnt[k] += 1
T = sum(tot.values())
print(f"# {sys.argv[2] if len(sys.argv) > 2 else 'launch list'}\n")
print("`ncu --metrics gpu__time_duration.sum --clock-control none -c 400 python bench.py --steps 300 --warmup 10 "
      "--no-cpu-baseline` (cold-cache, serialised: compare shares, not absolutes)\n")
print("| launches | total us | share | mean us | kernel |\n|---|---|---|---|---|")
for k, v in tot.most_common():
    print(f"| {cnt[k]} | {v:.1f} | {100 * v / T:.1f}% | {v / cnt[k]:.1f} | `{k}` |")
