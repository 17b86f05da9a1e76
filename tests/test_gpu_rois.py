"""GPU parity for multi-template / ROI matching (the paper's TM runtime
operation: several templates per frame, each searched inside its region of interest --
Tab 5.1 caption P:190-191, 5.1.3.4 P:91).  Reference: the oracle's full corr2 / SSD surface
of each (frame, template) restricted to the clipped ROI; peak = argmax (argmin for SSD)
inside it, tie -> smallest u*V+v."""
import numpy as np
import pytest
import torch

import oracle
import synth
from paper_conf_ipps_moorelk13_b200 import _native as N
from paper_conf_ipps_moorelk13_b200 import build as B
from paper_conf_ipps_moorelk13_b200.api import MatchPlan, decode_peaks

pytestmark = pytest.mark.gpu
TOL = 1e-4


@pytest.fixture(scope="module", autouse=True)
def _lib():
    B.build()


def make_case(H, W, h, w, T, F, rh, rw, seed):
    g = synth.rng(seed)
    imgs = np.stack([synth.uniform_image(H, W, seed + f) for f in range(F)])
    U, V = H - h + 1, W - w + 1
    tmpls, rois, plants = [], np.zeros((F, T, 2), np.int32), []
    for t in range(T):
        u0, v0 = int(g.integers(0, U)), int(g.integers(0, V))
        tmpls.append(imgs[t % F, u0:u0 + h, v0:v0 + w])
        plants.append((t % F, u0, v0))
    for f in range(F):
        for t in range(T):
            pf, pu, pv = plants[t]
            if pf == f:  # ROI around the plant (clipped at the valid range on purpose near borders)
                rois[f, t] = (max(0, pu - int(g.integers(0, rh))), max(0, pv - int(g.integers(0, rw))))
            else:
                rois[f, t] = (int(g.integers(0, U)), int(g.integers(0, V)))
    return imgs, np.ascontiguousarray(np.stack(tmpls)), rois, plants


@pytest.mark.parametrize("H,W,h,w,T,F,rh,rw,score", [
    (200, 180, 16, 16, 5, 2, 40, 56, N.NCC_SCORE_NCC),    # constant-bank templates (AOT 16x16)
    (260, 240, 33, 27, 3, 2, 48, 37, N.NCC_SCORE_NCC),    # run-time specialised, constant bank
    (300, 300, 64, 64, 6, 1, 64, 96, N.NCC_SCORE_NCC),    # 6 x 64 x 64 > 64 KB: shared-memory templates
    (200, 180, 16, 16, 4, 2, 40, 56, N.NCC_SCORE_SSD),
])
def test_rois_vs_oracle(H, W, h, w, T, F, rh, rw, score):
    imgs, tmpls, rois, plants = make_case(H, W, h, w, T, F, rh, rw, seed=h * 7 + T)
    dev = torch.device("cuda", 0)
    with MatchPlan(H, W, h, w, batch=F, n_templates=T, roi=(rh, rw), write_surface=True, score=score) as plan:
        pk, sc = plan.match_rois(torch.from_numpy(imgs).to(dev), torch.from_numpy(tmpls).to(dev),
                                 torch.from_numpy(rois).to(dev))
        torch.cuda.synchronize()
        info = plan.info.as_dict()
    d = {k: v.cpu().numpy().reshape(F, T) for k, v in decode_peaks(pk.reshape(-1, 4)).items()}
    sc = sc.cpu().numpy()
    U, V = H - h + 1, W - w + 1
    for f in range(F):
        for t in range(T):
            ref_full = oracle.ncc_surface(imgs[f], tmpls[t]) if score == N.NCC_SCORE_NCC else \
                oracle.ssd_surface(imgs[f], tmpls[t])
            u0, v0 = rois[f, t]
            u1, v1 = min(u0 + rh, U), min(v0 + rw, V)
            ref = ref_full[u0:u1, v0:v1]
            got = sc[f, t, :u1 - u0, :v1 - v0]
            tol = TOL if score == N.NCC_SCORE_NCC else 1e-5 * float(2 * (tmpls[t].astype(np.float64) ** 2).sum() + 10)
            assert np.max(np.abs(got - ref)) <= tol, (f, t, info["variant_name"])
            k = int(np.argmax(ref) if score == N.NCC_SCORE_NCC else np.argmin(ref))
            exp = (u0 + k // (v1 - v0), v0 + k % (v1 - v0))
            if plants[t][0] == f and u0 <= plants[t][1] < u1 and v0 <= plants[t][2] < v1:
                assert exp == (plants[t][1], plants[t][2])
                assert (int(d["u"][f, t]), int(d["v"][f, t])) == exp


def test_roi_plan_rejects_plain_match_and_bad_rois():
    with MatchPlan(128, 128, 16, 16, n_templates=2, roi=(8, 8)) as plan:
        with pytest.raises(N.NccError):
            plan.match(torch.zeros((1, 128, 128), device="cuda"), torch.zeros((16, 16), device="cuda"))
    with pytest.raises(N.NccError):
        MatchPlan(128, 128, 16, 16, n_templates=2, roi=(200, 8))


@pytest.mark.parametrize("H,W,h,w,T,F,rh,rw,score", [
    (200, 180, 16, 16, 5, 2, 40, 56, N.NCC_SCORE_NCC),
    (260, 240, 33, 27, 3, 2, 48, 37, N.NCC_SCORE_NCC),
    (300, 300, 64, 64, 6, 1, 64, 96, N.NCC_SCORE_NCC),
    (420, 400, 150, 140, 3, 2, 150, 260, N.NCC_SCORE_NCC),  # 2 x 5 template blocks, 3 column tiles
    (200, 180, 16, 16, 4, 2, 40, 56, N.NCC_SCORE_SSD),
])
def test_rois_on_tensor_cores_vs_oracle(H, W, h, w, T, F, rh, rw, score, monkeypatch):
    """ROI / multi-template matching on the tensor-core numerator (tcgen05 3xTF32, planes mode):
    every (frame, template) pair is a sub-problem whose ROI origin the kernel reads at run time;
    same checks as the CUDA-core path (clipped ROI surfaces within 1e-4, planted peaks exact)."""
    monkeypatch.setenv("NCC_TC", "1")
    with MatchPlan(H, W, h, w, batch=F, n_templates=T, roi=(rh, rw)) as plan:
        name = plan.info.variant_name.decode()
        assert name.startswith("tm_tc") and name.endswith("_roi"), name
    test_rois_vs_oracle(H, W, h, w, T, F, rh, rw, score)
