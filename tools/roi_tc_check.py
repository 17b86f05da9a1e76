"""One ROI match on the tensor-core path (debug aid): python tools/roi_tc_check.py"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ.setdefault("NCC_TC", "1")
import numpy as np  # noqa: E402
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_ipps_moorelk13_b200.api import MatchPlan, decode_peaks  # noqa: E402

H, W, h, w, T, F, rh, rw = 200, 180, 16, 16, 2, 1, 40, 56
imgs = np.stack([synth.uniform_image(H, W, 5 + f) for f in range(F)])
tm = np.ascontiguousarray(np.stack([imgs[0, 10:10 + h, 20:20 + w], imgs[0, 50:50 + h, 60:60 + w]]))
rois = np.array([[[5, 10], [40, 50]]], np.int32)
dev = torch.device("cuda", 0)
with MatchPlan(H, W, h, w, batch=F, n_templates=T, roi=(rh, rw), write_surface=True) as plan:
    print(plan.info.variant_name.decode(), flush=True)
    pk, sc = plan.match_rois(torch.from_numpy(imgs).to(dev), torch.from_numpy(tm).to(dev), torch.from_numpy(rois).to(dev))
    torch.cuda.synchronize()
    print(decode_peaks(pk.reshape(-1, 4)))
