#!/usr/bin/env python
"""Summarise ncu captures into profiles/ (committed evidence).

  python tools/ncu_summary.py full  <rep.ncu-rep> <out.json>     # one --set full capture
  python tools/ncu_summary.py launches <launches.csv> <out.json>  # gpu__time_duration list
"""
import csv
import io
import json
import subprocess
import sys
from collections import OrderedDict, defaultdict

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_bytes.sum",
        "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
        "launch__shared_mem_per_block_dynamic", "sm__cycles_elapsed.avg.per_second",
        "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active",
        "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
        "smsp__sass_thread_inst_executed_op_ffma_pred_on.sum", "smsp__inst_executed.sum",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "sm__cycles_active.avg", "gpc__cycles_elapsed.max",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum",
        "sm__pipe_tensor_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed",
        "sm__mem_tensor_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_uniform.avg.pct_of_peak_sustained_active"]


def full(rep, out):
    txt = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(txt)))
    h, u = rows[0], rows[1]
    res = []
    for v in rows[2:]:
        d = OrderedDict()
        d["kernel"] = v[h.index("Kernel Name")]
        for k in KEYS:
            if k in h:
                d[k] = {"value": v[h.index(k)], "unit": u[h.index(k)]}
        stalls = {n.replace("smsp__pcsamp_warps_issue_stalled_", ""): int(float(v[i] or 0))
                  for i, n in enumerate(h) if n.startswith("smsp__pcsamp_warps_issue_stalled_")
                  and not n.endswith("_not_issued")}
        d["stall_samples"] = dict(sorted(stalls.items(), key=lambda kv: -kv[1]))
        res.append(d)
    json.dump(res, open(out, "w"), indent=1)


def launches(path, out):
    rows = list(csv.reader(open(path)))
    hi = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    h = rows[hi]
    ki, vi = h.index("Kernel Name"), h.index("Metric Value")
    d = defaultdict(list)
    for r in rows[hi + 1:]:
        if len(r) > vi:
            d[r[ki]].append(float(r[vi].replace(",", "")))
    tot = sum(sum(v) for v in d.values())
    res = [{"kernel": k, "launches": len(v), "mean_ns": sum(v) / len(v), "share": sum(v) / tot}
           for k, v in sorted(d.items(), key=lambda kv: -sum(kv[1]))]
    json.dump({"note": "ncu --metrics gpu__time_duration.sum --clock-control none (cold-cache, serialised)",
               "kernels": res}, open(out, "w"), indent=1)


if __name__ == "__main__":
    {"full": full, "launches": launches}[sys.argv[1]](sys.argv[2], sys.argv[3])
