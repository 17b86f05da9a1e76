#!/usr/bin/env python
"""Numerator error of the TM paths on the cancellation-stress input (SURVEY 8(d) smooth) against
the fp64 FFT route, per path / knob: max |dNCC|, where, and the brute-force oracle there.
Usage: python tools/tc_error.py [cfg] [smooth 0/1]"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import synth  # noqa: E402
from oracle.ncc_fft import ncc_surface_fft  # noqa: E402
from paper_conf_ipps_moorelk13_b200.api import MatchPlan  # noqa: E402

cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 5
smooth = bool(int(sys.argv[2])) if len(sys.argv) > 2 else True
c = synth.CONFIGS[cfg]
img, T, u0, v0 = synth.tm_inputs(cfg, k=3, smooth=smooth)
f = ncc_surface_fft(img, T)
dev = torch.device("cuda", 0)
d_img, d_t = torch.from_numpy(img).to(dev), torch.from_numpy(T).to(dev)
for name, env, kw in [("tc", {}, {}), ("tc_center", {"NCC_TC_CENTER": "1"}, {}),
                      ("tc_wc64", {"NCC_TC_WC": "64"}, {}), ("tc_wc64_center", {"NCC_TC_WC": "64", "NCC_TC_CENTER": "1"}, {}),
                      ("cuda_cores", {}, {"cuda_cores": True})]:
    for k in ("NCC_TC_CENTER", "NCC_TC_WC"):
        os.environ.pop(k, None)
    os.environ.update(env)
    with MatchPlan(c["H"], c["W"], c["h"], c["w"], write_surface=True, **kw) as plan:
        _, s = plan.match(d_img, d_t)
        torch.cuda.synchronize()
        s = s[0].cpu().numpy()
        var = plan.info.variant_name.decode()
    e = np.abs(s - f)
    k = int(np.argmax(e))
    u, v = divmod(k, s.shape[1])
    bf = float(oracle.ncc_at(img, T, [u], [v])[0])
    print(json.dumps({"path": name, "variant": var, "max_err": float(e.max()), "p99_err": float(np.quantile(e, 0.99)),
                      "at": [u, v], "gpu": float(s[u, v]), "fft": float(f[u, v]), "bruteforce": bf}), flush=True)
