"""Join the ncu launch list of tools/launch_cost_ncu.py with its printed launch order.

    python tools/launch_cost_join.py X.csv order.txt

Every printed line is one measured launch; flush kernels (torch fills) and torch's
random-number / conversion kernels are dropped by name.  Prints the median duration per tag.
"""
import collections
import csv
import statistics
import sys

rows = [r for r in csv.reader(open(sys.argv[1])) if r]
i = [k for k, r in enumerate(rows) if r and r[0] == "ID"][0]
hdr = rows[i]
kern = collections.OrderedDict()
for r in rows[i + 1:]:
    x = dict(zip(hdr, r))
    if x.get("Metric Name") != "gpu__time_duration.sum":
        continue
    kern[x["ID"]] = (x["Kernel Name"], float(x["Metric Value"]), x.get("Metric Unit", ""))
SKIP = ("vectorized_elementwise_kernel", "elementwise_kernel", "distribution", "fill", "unrolled_elementwise")
meas = [(n, v, u) for n, v, u in kern.values() if not any(s in n for s in SKIP)]
tags = [ln.rstrip("\n") for ln in open(sys.argv[2]) if ln.strip()]
if len(meas) != len(tags):
    print(f"warning: {len(meas)} kernels vs {len(tags)} tags", file=sys.stderr)
by = collections.OrderedDict()
for (n, v, u), t in zip(meas, tags):
    scale = 1e-3 if u in ("nsecond", "ns") else (1.0 if u in ("usecond", "us") else 1e3)
    by.setdefault(t, []).append((v * scale, n.split("(")[0][:50]))
for t, vs in by.items():
    print(f"{t:75s} {statistics.median(v for v, _ in vs):8.2f} us  {vs[0][1]}")
