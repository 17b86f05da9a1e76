"""Run a few PIV calls of cfg N with P pairs (profiling helper)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
import synth  # noqa: E402
from paper_conf_ipps_moorelk13_b200.api import PivPlan  # noqa: E402

cfg, P = int(sys.argv[1]), int(sys.argv[2])
if cfg == 3:
    P = 1  # cfg3 is one 1024 x 1024 pair (the repeats below are the launches)
c = synth.CONFIGS[cfg]
wl = dict(cfg=cfg, H=c["H"], W=c["W"], h=c["h"], w=c["w"], m=c["m"], step=c["step"], pairs=P, rank=0)
dev = torch.device("cuda", 0)
A, B, _ = bench.piv_frames_device(wl, dev, torch)
with PivPlan(c["H"], c["W"], c["h"], c["m"], c["step"], pairs=P) as plan:
    for _ in range(4):
        plan.correlate(A, B)
    torch.cuda.synchronize()
print("ok")
