"""Run one TM config a few times (for ncu captures): python tools/tm_one.py CFG [reps]."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_ipps_moorelk13_b200.api import MatchPlan  # noqa: E402

cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 2
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
c = synth.CONFIGS[cfg]
img, T, _, _ = synth.tm_inputs(cfg)
dev = torch.device("cuda", 0)
d_img, d_t = torch.from_numpy(img).to(dev), torch.from_numpy(T).to(dev)
with MatchPlan(c["H"], c["W"], c["h"], c["w"]) as plan:
    print(plan.info.variant_name.decode(), flush=True)
    for _ in range(reps):
        plan.match(d_img, d_t)
    torch.cuda.synchronize()
