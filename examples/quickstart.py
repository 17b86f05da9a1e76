"""Quick start: the README example (template match + PIV through the Python binding)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch
from paper_conf_ipps_moorelk13_b200.api import MatchPlan, PivPlan, decode_peaks, decode_vectors

img = torch.rand(1, 1024, 1024, device="cuda")            # frames (batch, H, W), fp32
tmpl = img[0, 300:428, 500:628].contiguous()               # 128 x 128 template
with MatchPlan(1024, 1024, 128, 128, write_surface=True) as plan:
    peaks, surface = plan.match(img, tmpl)                 # stream-ordered; graph replay after the 1st call
    print(decode_peaks(peaks))                             # score, u, v, flags per frame

A = torch.rand(4, 1024, 1024, device="cuda"); B = torch.roll(A, (3, -5), (1, 2))
with PivPlan(1024, 1024, win=32, search=16, step=16, pairs=4) as plan:
    vectors, _ = plan.correlate(A, B)                      # (pairs, Ky, Kx) vectors, sub-pixel dy/dx
    print(decode_vectors(vectors)["iy"][0, 10, 10])        # -> 3

