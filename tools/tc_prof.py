#!/usr/bin/env python
"""Per-CTA wait accounting of tm_tc_kernel (NCC_TC_EXP=32): run one TM config, dump the
[ticket][8] globaltimer record (start, end, epilogue flag wait, epilogue group wait, drain,
chain work, MMA drained wait, MMA a_full wait) and summarise it per template block.
Usage: python tools/tc_prof.py [cfg]"""
import json
import os
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 2
dump = os.path.join(tempfile.gettempdir(), f"tc_prof_{os.getpid()}.bin")
os.environ["NCC_TC_EXP"] = str(32 | int(os.environ.get("EXTRA_EXP", "0")))
os.environ["NCC_TC_PROF_DUMP"] = dump
import synth  # noqa: E402
from paper_conf_ipps_moorelk13_b200.api import MatchPlan  # noqa: E402

c = synth.CONFIGS[cfg]
img, T, _, _ = synth.tm_inputs(cfg)
dev = torch.device("cuda", 0)
d_img, d_t = torch.from_numpy(img).to(dev), torch.from_numpy(T).to(dev)
with MatchPlan(c["H"], c["W"], c["h"], c["w"]) as plan:
    for _ in range(4):
        plan.match(d_img, d_t)
    torch.cuda.synchronize()
    name = plan.info.variant_name.decode()
    nblk = plan.info.split
raw = np.fromfile(dump, dtype=np.uint64).astype(np.int64)
trace = raw[-512:].reshape(2, 4, 64)  # [chain done | MMA group commit][ticket][group]
r = raw[:-512].reshape(-1, 8)
t0 = r[:, 0].min()
out = {"variant": name, "ctas": len(r), "kernel_us": float((r[:, 1].max() - t0) / 1e3)}
fields = ["start", "end", "chain_flag_wait", "chain_staged_wait", "cta_end", "chain_work", "mma_drained_wait",
          "mma_afull_wait"]
per = {}
for b in range(nblk):
    rb = r[b::nblk]
    d = {"start_us": float((rb[:, 0] - t0).mean() / 1e3), "end_us": float((rb[:, 1] - t0).mean() / 1e3),
         "end_max_us": float((rb[:, 1] - t0).max() / 1e3)}
    for i, f in enumerate(fields[2:], 2):
        d[f + "_us"] = float(((rb[:, i] - t0) if f == "cta_end" else rb[:, i]).mean() / 1e3)
    per[f"blk{b}"] = d
out["per_block"] = per
out["trace_tile0"] = {f"blk{b}": {"mma_commit_us": [round((x - t0) / 1e3, 1) if x else None for x in trace[1, b]],
                                  "chain_done_us": [round((x - t0) / 1e3, 1) if x else None for x in trace[0, b]]}
                      for b in range(min(4, nblk))}
print(json.dumps(out, indent=1))
os.remove(dump)
