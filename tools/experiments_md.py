#!/usr/bin/env python
"""Regenerate the tables of EXPERIMENTS.md from profiles/r02_paper_sweeps.jsonl (the output of
tools/paper_sweeps.py): every '| ... |' table block that follows a '## Tab ...' heading is
replaced; headings and prose stay.  Usage: python tools/experiments_md.py [jsonl] [md]"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def fmt(x):
    if isinstance(x, float):
        return f"{x:.3g}" if abs(x) < 1e4 else f"{x:.3g}"
    return str(x)


def tables(rows):
    out = {}
    tm = [r for r in rows if r["table"] == "6.13"]
    out["6.13"] = ["| cfg | tier | variant | regs/thread | numerator ms | step ms | TFLOP/s | correct |",
                   "|---|---|---|---|---|---|---|---|"] + [
        f"| {r['cfg']} | {r['tier']} | {r['variant']} | {r['regs']} | {fmt(r['numerator_ms'])} | {fmt(r['step_ms'])} | "
        f"{r['tflops']:.1f} | {r['correct']} |" for r in tm]
    odd = [r for r in rows if r["table"] == "5.2"]
    for r in odd:  # the default plan of an unmatched shape may take the tensor-core numerator
        if r["variant"].startswith("tm_tc"):
            r["tier"] = "TC"
    out["5.2"] = ["| tier | variant | regs | numerator ms | TFLOP/s | correct |", "|---|---|---|---|---|---|"] + [
        f"| {r['tier']} | {r['variant']} | {r['regs']} | {fmt(r['numerator_ms'])} | {r['tflops']:.1f} | {r['correct']} |"
        for r in odd]
    for t in ("6.16", "6.17", "6.18"):
        pv = [r for r in rows if r["table"] == t]
        out[t] = ["| mask | m | step | tier | variant | regs | vectors | vectors/s | numerator TFLOP/s | correct |",
                  "|---|---|---|---|---|---|---|---|---|---|"] + [
            f"| {r['win']} | {r['m']} | {r['step']} | {r['tier']} | {r['variant']} | {r['regs']} | {r['vectors']} | "
            f"{r['vectors_per_s']:.3g} | {r['tflops']:.3g} | {r['correct']} |" for r in pv]
    return out


def main():
    src = sys.argv[1] if len(sys.argv) > 1 else os.path.join(ROOT, "profiles", "r02_paper_sweeps.jsonl")
    md = sys.argv[2] if len(sys.argv) > 2 else os.path.join(ROOT, "EXPERIMENTS.md")
    rows = [json.loads(l) for l in open(src) if l.strip().startswith("{")]
    tabs = tables(rows)
    key_of = {"Tab 6.13": "6.13", "Tab 5.2": "5.2", "Tab 6.4 / 6.16": "6.16", "Tab 6.5 / 6.17": "6.17",
              "Tab 6.6 / 6.18": "6.18"}
    lines = open(md).read().split("\n")
    out, cur, i = [], None, 0
    while i < len(lines):
        ln = lines[i]
        if ln.startswith("## "):
            cur = next((v for k, v in key_of.items() if ln.startswith("## " + k)), None)
        if cur and ln.startswith("|"):
            while i < len(lines) and lines[i].startswith("|"):
                i += 1
            out.extend(tabs[cur])
            cur = None
            continue
        out.append(ln)
        i += 1
    open(md, "w").write("\n".join(out))


if __name__ == "__main__":
    main()
