"""Debug helper: ROI cases with explicit origins: args H W h w T F rh rw then u,v pairs."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_ipps_moorelk13_b200.api import MatchPlan
import synth
H, W, h, w, T, F, rh, rw = map(int, sys.argv[1:9])
o = list(map(int, sys.argv[9:]))
rois = np.array(o, np.int32).reshape(F, T, 2)
imgs = np.stack([synth.uniform_image(H, W, 5 + f) for f in range(F)])
tm = np.ascontiguousarray(np.stack([imgs[0, :h, :w]] * T))
dev = torch.device("cuda", 0)
with MatchPlan(H, W, h, w, batch=F, n_templates=T, roi=(rh, rw), write_surface=True) as plan:
    pk, sc = plan.match_rois(torch.from_numpy(imgs).to(dev), torch.from_numpy(tm).to(dev), torch.from_numpy(rois).to(dev))
    torch.cuda.synchronize()
print("ok", pk.cpu().tolist())
