"""The tensor-core TM path's alternative block combinations and launch schedules compute the
same numbers bit for bit: planes mode (per-block partial planes summed by
tm_tc_finish) and chain mode (blocks chained inside tm_tc_kernel) both form ((p0 + p1) + p2) + ...
per output and normalise with the same fp32 factors; schedules 0 / 3 / 4 / 5 only reorder the
launches.  Checked on shapes with 1-20 template blocks, ragged last columns, batches, SSD, and
against the fp64 oracle."""
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


def run(imgs, T, score=N.NCC_SCORE_NCC):
    F, H, W = imgs.shape
    h, w = T.shape
    dev = torch.device("cuda", 0)
    with MatchPlan(H, W, h, w, batch=F, write_surface=True, score=score) as plan:
        pk, s = plan.match(torch.from_numpy(imgs).to(dev), torch.from_numpy(np.ascontiguousarray(T)).to(dev))
        torch.cuda.synchronize()
        name = plan.info.variant_name.decode()
    return pk.cpu().numpy(), s.cpu().numpy(), name


@pytest.mark.parametrize("H,W,h,w,F,smooth,score", [
    (330, 290, 40, 36, 2, False, N.NCC_SCORE_NCC),      # 2 blocks (36 = 32 + 4 columns)
    (400, 556, 300, 300, 1, False, N.NCC_SCORE_NCC),    # 3 x 10 = 30 blocks, ragged column kernel
    (1024, 1024, 128, 128, 1, True, N.NCC_SCORE_NCC),   # cfg2 smooth: 4 blocks
    (300, 330, 140, 70, 2, False, N.NCC_SCORE_SSD),     # SSD, 2 x 3 blocks
])
def test_planes_and_chain_modes_bitwise_equal(H, W, h, w, F, smooth, score, monkeypatch):
    monkeypatch.setenv("NCC_TC", "1")
    imgs = np.stack([(synth.smooth_image if smooth else synth.uniform_image)(H, W, 800 + k) for k in range(F)])
    T, u0, v0 = synth.planted_template(imgs[-1], h, w, 801)
    out = {}
    for mode in ("1", "0"):
        monkeypatch.setenv("NCC_TC_PLANES", mode)
        out[mode] = run(imgs, T, score)
        assert ("_planes" if mode == "1" else "_chain") in out[mode][2], out[mode][2]
    np.testing.assert_array_equal(out["1"][1], out["0"][1])
    np.testing.assert_array_equal(out["1"][0], out["0"][0])
    d = decode_peaks(torch.from_numpy(out["0"][0]))
    assert (int(d["u"][F - 1]), int(d["v"][F - 1])) == (u0, v0)
    g = synth.rng(802)
    U, V = H - h + 1, W - w + 1
    us, vs = g.integers(0, U, 60), g.integers(0, V, 60)
    vs[:4] = V - 1  # the ragged last column
    ref = oracle.ncc_at(imgs[-1], T, us, vs) if score == N.NCC_SCORE_NCC else \
        np.array([float(((T.astype(np.float64) - imgs[-1][u:u + h, v:v + w]) ** 2).sum()) for u, v in zip(us, vs)])
    tol = TOL if score == N.NCC_SCORE_NCC else 1e-5 * float(2 * (T.astype(np.float64) ** 2).sum() + 10)
    assert np.max(np.abs(out["0"][1][F - 1][us, vs] - ref)) <= tol


@pytest.mark.parametrize("sched", ["0", "4", "5"])
def test_launch_schedules_bitwise_equal(sched, monkeypatch):
    img, T, u0, v0 = synth.tm_inputs(2, k=31)
    imgs = img[None]
    base = run(imgs, T)
    monkeypatch.setenv("NCC_TM_SCHED", sched)
    alt = run(imgs, T)
    assert base[2].startswith("tm_tc")
    np.testing.assert_array_equal(alt[1], base[1])
    np.testing.assert_array_equal(alt[0], base[0])
