#!/usr/bin/env python
"""Render the Tab 6.21 / 6.22 sensitivity surfaces (tools/sensitivity.py output) as "% of best"
tables into EXPERIMENTS.md, replacing the table block under each '## Tab 6.21' / '## Tab 6.22'
heading (appending the sections if missing).  Usage: python tools/sensitivity_md.py [jsonl] [md]"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

HEAD = {
    "6.21": ("## Tab 6.21 analogue — TM: % of best over main tile size x threads per block",
             "Paper: 'Template matching: percentage of peak performance ... main tile size ... threads' (P:236-237). "
             "Run-time specialised (NVRTC) CUDA-core numerator kernels on cfg2 (1024^2 image, 128^2 template); "
             "tile = 8 WY output rows x 4 RV WX output columns, threads = 32 WX WY; cell = % of the best "
             "configuration's numerator TFLOP/s (best = 100), `--` = not built (TMA box limit or compile). "
             "Every point found the planted peak."),
    "6.22": ("## Tab 6.22 analogue — PIV: % of best over data registers x threads per block",
             "Paper: 'PIV: percentage of peak performance ... data registers ... threads' (P:238-240). "
             "Run-time specialised PIV kernels on cfg3 (1024^2 pair, 32^2 masks, +-16, step 16); data registers "
             "RV = offsets held per thread, threads = WPB windows per block x ceil(items/32) warps; cell = % of the "
             "best point (threads in parentheses).  Every point recovered the planted shift in all windows."),
}


def surfaces(rows):
    out = {}
    tm = [r for r in rows if r["table"] == "6.21" and "tflops" in r]
    if tm:
        best = max(r["tflops"] for r in tm)
        cols = sorted({(r["tile_rows"], r["WX"], r["WY"]) for r in tm}, key=lambda c: (32 * c[1] * c[2], c[0]))
        hdr = "| RV (cols/lane) | " + " | ".join(f"{32 * wx * wy} thr, {8 * wy} rows x {wx} col-warps" for _, wx, wy in cols) + " |"
        lines = [hdr, "|---" * (len(cols) + 1) + "|"]
        for rv in sorted({r["RV"] for r in tm}):
            cells = []
            for (_, wx, wy) in cols:
                m = [r for r in tm if r["RV"] == rv and r["WX"] == wx and r["WY"] == wy]
                cells.append(f"{100 * m[0]['tflops'] / best:.0f} ({m[0]['tile_rows']}x{m[0]['tile_cols']})" if m else "--")
            lines.append(f"| {rv} | " + " | ".join(cells) + " |")
        b = max(tm, key=lambda r: r["tflops"])
        lines.append("")
        lines.append(f"Best: RV {b['RV']}, {b['threads']} threads, tile {b['tile_rows']}x{b['tile_cols']}: "
                     f"{b['tflops']:.1f} TFLOP/s ({b['regs']} regs/thread).")
        out["6.21"] = lines
    pv = [r for r in rows if r["table"] == "6.22" and "tflops" in r]
    if pv:
        best = max(r["tflops"] for r in pv)
        wpbs = sorted({r["WPB"] for r in pv})
        lines = ["| RV (data registers) | " + " | ".join(f"{w} window(s)/block" for w in wpbs) + " |",
                 "|---" * (len(wpbs) + 1) + "|"]
        for rv in sorted({r["RV"] for r in pv}):
            cells = []
            for w in wpbs:
                m = [r for r in pv if r["RV"] == rv and r["WPB"] == w]
                cells.append(f"{100 * m[0]['tflops'] / best:.0f} ({m[0]['threads']})" if m else "--")
            lines.append(f"| {rv} | " + " | ".join(cells) + " |")
        b = max(pv, key=lambda r: r["tflops"])
        lines.append("")
        lines.append(f"Best: RV {b['RV']}, {b['threads']} threads ({b['WPB']} window/block): {b['tflops']:.1f} TFLOP/s "
                     f"({b['regs']} regs/thread); the default cfg3 kernel (persistent warp-specialised piv_ws2, "
                     f"DESIGN.md 6.1) is not in this grid.")
        out["6.22"] = lines
    return out


def main():
    src = sys.argv[1] if len(sys.argv) > 1 else os.path.join(ROOT, "profiles", "r02_sensitivity.jsonl")
    md = sys.argv[2] if len(sys.argv) > 2 else os.path.join(ROOT, "EXPERIMENTS.md")
    rows = [json.loads(l) for l in open(src) if l.strip().startswith("{")]
    tabs = surfaces(rows)
    text = open(md).read()
    for key, lines in tabs.items():
        head, prose = HEAD[key]
        block = head + "\n\n" + prose + "\n\n" + "\n".join(lines) + "\n"
        if head in text:
            i = text.index(head)
            j = text.find("\n## ", i + len(head))
            text = text[:i] + block + ("\n" + text[j + 1:] if j >= 0 else "")
        else:
            text = text.rstrip("\n") + "\n\n" + block
    open(md, "w").write(text)


if __name__ == "__main__":
    main()
