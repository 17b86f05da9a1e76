#!/usr/bin/env python
"""Split ncu source-page stall samples of one kernel into code regions.

  python tools/ncu_regions.py <rep.ncu-rep>
Regions are contiguous address ranges delimited by the first/last FFMA2 (consumer core loop),
reported with the per-reason stall samples and instruction counts of each region.
"""
import csv
import io
import subprocess
import sys
from collections import Counter

rep = sys.argv[1]
txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(txt)))
hdr, data = rows[1], rows[2:]
isrc = hdr.index("Source")
iall = hdr.index("Warp Stall Sampling (All Samples)")
iex = hdr.index("Instructions Executed")
sc = [(i, h[6:]) for i, h in enumerate(hdr) if h.startswith("stall_") and "Not Issued" not in h]
ops = [r[isrc].split()[0] if r[isrc].split() and not r[isrc].split()[0].startswith("@") else
       (r[isrc].split()[1] if len(r[isrc].split()) > 1 else "") for r in data]
ff = [k for k, o in enumerate(ops) if o.startswith("FFMA2")]
lo, hi = (ff[0] - 80, ff[-1] + 20) if ff else (0, -1)
regions = {"core": range(max(lo, 0), hi + 1)}
tot = Counter()
for name, rg in list(regions.items()) + [("rest", [k for k in range(len(data)) if not (lo <= k <= hi)])]:
    c = Counter()
    ninst = 0
    opc = Counter()
    for k in rg:
        r = data[k]
        for i, h in sc:
            c[h] += int(float(r[i] or 0))
        n = int(float(r[iex] or 0))
        ninst += n
        opc[ops[k].split(".")[0]] += n
    s = sum(c.values())
    print(f"== {name}: samples {s}, warp-instructions {ninst}")
    print("   stalls:", ", ".join(f"{h} {v} ({100 * v / max(s, 1):.0f}%)" for h, v in c.most_common(8)))
    print("   ops:", ", ".join(f"{o} {v}" for o, v in opc.most_common(8)))

if len(sys.argv) > 2:  # top instructions by samples outside the core loop
    top = int(sys.argv[2])
    rest = [(int(float(data[k][iall] or 0)), k) for k in range(len(data)) if not (lo <= k <= hi)]
    rest.sort(reverse=True)
    print(f"== top {top} sampled instructions outside the core loop (index, samples, reasons, source)")
    for smp, k in rest[:top]:
        r = data[k]
        rs = sorted(((int(float(r[i] or 0)), h) for i, h in sc), reverse=True)[:3]
        print(f"{k:6d} {smp:7d}  {', '.join(f'{h}:{v}' for v, h in rs if v):50s} {r[isrc][:70]}")
