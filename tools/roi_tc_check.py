"""ROI matches on the tensor-core path (debug aid): python tools/roi_tc_check.py T F [seed]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
os.environ.setdefault("NCC_TC", "1")
import torch  # noqa: E402

from test_gpu_rois import make_case  # noqa: E402
from paper_conf_ipps_moorelk13_b200.api import MatchPlan, decode_peaks  # noqa: E402

T, F = int(sys.argv[1]), int(sys.argv[2])
seed = int(sys.argv[3]) if len(sys.argv) > 3 else 117
H, W, h, w, rh, rw = 200, 180, 16, 16, 40, 56
imgs, tm, rois, plants = make_case(H, W, h, w, T, F, rh, rw, seed)
if os.environ.get("ROI_X") is not None:  # force every ROI's column origin
    rois[..., 1] = int(os.environ["ROI_X"])
dev = torch.device("cuda", 0)
with MatchPlan(H, W, h, w, batch=F, n_templates=T, roi=(rh, rw), write_surface=True) as plan:
    print(T, F, plan.info.variant_name.decode(), rois.tolist(), flush=True)
    pk, sc = plan.match_rois(torch.from_numpy(imgs).to(dev), torch.from_numpy(tm).to(dev), torch.from_numpy(rois).to(dev))
    torch.cuda.synchronize()
    print("ok", decode_peaks(pk.reshape(-1, 4))["u"].tolist(), flush=True)
