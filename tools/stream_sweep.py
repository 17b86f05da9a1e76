#!/usr/bin/env python
"""TM host-path streaming: 8 frames of cfg2 per call through ncc_match_host with chunk sizes
1/2/4/8 frames (NCC_TM_CHUNK), against the device-resident 8-frame batch.  Prints JSON lines."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_ipps_moorelk13_b200.api import MatchPlan  # noqa: E402

img, T, _, _ = synth.tm_inputs(2)
F = 8
dev = torch.device("cuda", 0)
imgs = np.ascontiguousarray(np.broadcast_to(img, (F,) + img.shape))
hi, ht = torch.from_numpy(imgs).pin_memory(), torch.from_numpy(T).pin_memory()
di, dt = hi.to(dev), ht.to(dev)
hp = torch.empty((F, 4), dtype=torch.int32).pin_memory()


def timed(fn, n=10):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(n):
        fn()
    e1.record()
    e1.synchronize()
    return e0.elapsed_time(e1) / n


with MatchPlan(1024, 1024, 128, 128, batch=F) as plan:
    dev_ms = timed(lambda: plan.match(di, dt))
print(json.dumps({"path": "device", "frames": F, "ms": dev_ms}), flush=True)
for ch in ("1", "2", "4", "8"):
    os.environ["NCC_TM_CHUNK"] = ch
    with MatchPlan(1024, 1024, 128, 128, batch=F) as plan:
        ms = timed(lambda: plan.match_host(hi, ht, hp))
    print(json.dumps({"path": "host_stream", "chunk": int(ch), "ms": ms, "frac_of_device": dev_ms / ms}), flush=True)
