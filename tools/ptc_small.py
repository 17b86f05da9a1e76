"""Debug helper: one PIV call on the tensor-core path (H W h m step [pairs])."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_ipps_moorelk13_b200.api import PivPlan  # noqa: E402

H, W, h, m, step = (int(x) for x in sys.argv[1:6])
P = int(sys.argv[6]) if len(sys.argv) > 6 else 1
p = synth.particle_pair_integer(H, W, 2, -3, seed=1)
dev = torch.device("cuda", 0)
A = torch.from_numpy(p.A[None].copy()).to(dev).expand(P, H, W).contiguous()
B = torch.from_numpy(p.B[None].copy()).to(dev).expand(P, H, W).contiguous()
with PivPlan(H, W, h, m, step, pairs=P) as plan:
    v, sc = plan.correlate(A, B, scores=True)
    torch.cuda.synchronize()
    print(plan.info.as_dict()["variant_name"])
print("ok")
