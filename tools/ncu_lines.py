#!/usr/bin/env python
"""Per-CUDA-source-line stall samples of one kernel in an ncu report (--import-source on).

  python tools/ncu_lines.py <rep.ncu-rep> <function substring> [top N]
Prints the lines with the most warp-stall samples: samples, top stall reasons, instructions
executed, and the source text.
"""
import csv
import io
import subprocess
import sys
from collections import Counter, defaultdict


def main():
    rep, fn = sys.argv[1], sys.argv[2]
    top = int(sys.argv[3]) if len(sys.argv) > 3 else 30
    txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(txt)))
    cur_fn, cur_file, hdr = None, None, None
    samples, reasons, insts, src = Counter(), defaultdict(Counter), Counter(), {}
    line = None
    for r in rows:
        if not r:
            continue
        if r[0] == "File Path":
            cur_file = r[1].split("/")[-1]
            continue
        if r[0] == "Function Name":
            cur_fn = r[1]
            continue
        if r[0] == "Line No":
            hdr = r
            continue
        if hdr is None or cur_fn is None or fn not in cur_fn:
            continue
        d = dict(zip(hdr, r))
        if d.get("Line No"):
            line = (cur_file, int(d["Line No"]))
            src[line] = d.get("Source", "")[:110] if hdr.index("Source") == 1 else src.get(line, "")
        if line is None:
            continue
        try:
            s = int(float(d.get("Warp Stall Sampling (All Samples)") or 0))
        except ValueError:
            s = 0
        samples[line] += s
        try:
            insts[line] += int(float(d.get("Instructions Executed") or 0))
        except ValueError:
            pass
        for k, v in d.items():
            if k.startswith("stall_") and "Not Issued" not in k:
                try:
                    reasons[line][k[6:]] += int(float(v or 0))
                except ValueError:
                    pass
    tot = sum(samples.values()) or 1
    print(f"total samples {tot}")
    for ln, s in samples.most_common(top):
        rs = ", ".join(f"{k} {v}" for k, v in reasons[ln].most_common(3) if v)
        print(f"{s:8d} {100.0 * s / tot:5.1f}%  {ln[0]}:{ln[1]:<5d} inst {insts[ln]:>11d}  [{rs}]  {src.get(ln, '').strip()}")


if __name__ == "__main__":
    main()
