#!/usr/bin/env python
"""Run-to-run determinism of the tensor-core TM path: the same match N times (fresh plans and
repeated calls), surfaces compared bit for bit, plus the max |dNCC| against the fp64 FFT route.
Usage: python tools/tc_determinism.py [cfg] [smooth] [runs]"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import synth  # noqa: E402
from oracle.ncc_fft import ncc_surface_fft  # noqa: E402
from paper_conf_ipps_moorelk13_b200.api import MatchPlan  # noqa: E402

cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 5
smooth = bool(int(sys.argv[2])) if len(sys.argv) > 2 else True
runs = int(sys.argv[3]) if len(sys.argv) > 3 else 4
c = synth.CONFIGS[cfg]
img, T, u0, v0 = synth.tm_inputs(cfg, k=3, smooth=smooth)
f = ncc_surface_fft(img, T)
dev = torch.device("cuda", 0)
d_img, d_t = torch.from_numpy(img).to(dev), torch.from_numpy(T).to(dev)
ref = None
for r in range(runs):
    with MatchPlan(c["H"], c["W"], c["h"], c["w"], write_surface=True) as plan:
        for rep in range(2):
            _, s = plan.match(d_img, d_t)
            torch.cuda.synchronize()
            s = s[0].cpu().numpy()
            same = None if ref is None else bool(np.array_equal(s, ref))
            ndiff = None if ref is None else int((s != ref).sum())
            if ref is None:
                ref = s.copy()
            e = np.abs(s - f)
            k = int(np.argmax(e))
            print(json.dumps({"run": r, "rep": rep, "variant": plan.info.variant_name.decode(), "bitwise_same": same,
                              "ndiff": ndiff, "max_err": float(e.max()), "at": list(divmod(k, s.shape[1]))}), flush=True)
