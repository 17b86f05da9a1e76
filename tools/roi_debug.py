"""Debug helper: run one ROI case (args: H W h w T F rh rw score) and print the outcome."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
from test_gpu_rois import make_case
from paper_conf_ipps_moorelk13_b200.api import MatchPlan
H, W, h, w, T, F, rh, rw, score = map(int, sys.argv[1:10])
imgs, tmpls, rois, plants = make_case(H, W, h, w, T, F, rh, rw, seed=h * 7 + T)
print("rois", rois.tolist(), flush=True)
dev = torch.device("cuda", 0)
with MatchPlan(H, W, h, w, batch=F, n_templates=T, roi=(rh, rw), write_surface=True, score=score) as plan:
    print(plan.info.as_dict(), flush=True)
    pk, sc = plan.match_rois(torch.from_numpy(imgs).to(dev), torch.from_numpy(tmpls).to(dev),
                             torch.from_numpy(rois).to(dev))
    torch.cuda.synchronize()
print("ok", pk.cpu().tolist())
