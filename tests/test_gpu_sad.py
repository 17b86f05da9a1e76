"""GPU parity for the SAD score (sum |T - W|; the metric of the paper's Ch. 4 specialisation
example) through the C ABI vs the fp64 oracle: TM surfaces and argmin peaks, PIV
vectors and window surfaces.

Tolerance (derived): the GPU sums |t - b| in fp32 with a fresh partial per template
row, so |dSAD| <= 1e-5 * (sum|T| + sum|W|) per offset (the energy-scale bound used for SSD, with
the L1 norm in place of the squared one).
"""
import numpy as np
import pytest
import torch

import oracle
import synth
from paper_conf_ipps_moorelk13_b200 import _native as N
from paper_conf_ipps_moorelk13_b200 import build as B
from paper_conf_ipps_moorelk13_b200.api import MatchPlan, PivPlan, decode_peaks, decode_vectors

pytestmark = pytest.mark.gpu
REL = 1e-5


@pytest.fixture(scope="module", autouse=True)
def _lib():
    B.build()


def l1_scale(img, T):
    from oracle.ncc_fft import window_sums
    S1, _ = window_sums(np.abs(img), *T.shape)  # sum |W| per window
    return float(np.abs(T.astype(np.float64)).sum()) + S1


@pytest.mark.parametrize("H,W,h,w", [(64, 64, 16, 16), (150, 203, 37, 29), (300, 280, 130, 70)])
def test_tm_sad_surface_and_argmin(H, W, h, w):
    img = synth.uniform_image(H, W, 500 + h)
    T, u0, v0 = synth.planted_template(img, h, w, 501 + w)
    ref, pk = oracle.sad_match(img, T)
    dev = torch.device("cuda", 0)
    with MatchPlan(H, W, h, w, write_surface=True, score=N.NCC_SCORE_SAD) as plan:
        assert plan.info.variant_name.decode().startswith("tm_sad")
        peaks, s = plan.match(torch.from_numpy(img).to(dev), torch.from_numpy(T).to(dev))
        torch.cuda.synchronize()
    s = s[0].cpu().numpy()
    assert np.all(np.abs(s - ref) <= REL * l1_scale(img, T))
    d = decode_peaks(peaks)
    assert (int(d["u"][0]), int(d["v"][0])) == (u0, v0) == (pk.u, pk.v)
    assert abs(float(d["score"][0])) <= REL * float(l1_scale(img, T)[u0, v0]) and int(d["flags"][0]) == 0


def test_tm_sad_batch_band_and_host_path():
    imgs = np.stack([synth.uniform_image(120, 140, 510 + k) for k in range(3)])
    T, u0, v0 = synth.planted_template(imgs[2], 20, 24, 513)
    dev = torch.device("cuda", 0)
    with MatchPlan(120, 140, 20, 24, batch=3, write_surface=True, score=N.NCC_SCORE_SAD) as plan:
        pk, s = plan.match(torch.from_numpy(imgs).to(dev), torch.from_numpy(T).to(dev))
        hp = torch.empty((3, 4), dtype=torch.int32).pin_memory()
        plan.match_host(torch.from_numpy(imgs).pin_memory(), torch.from_numpy(T).pin_memory(), hp)
        torch.cuda.synchronize()
    np.testing.assert_array_equal(hp.numpy(), pk.cpu().numpy())
    for k in range(3):
        ref = oracle.sad_surface(imgs[k], T)
        assert np.all(np.abs(s[k].cpu().numpy() - ref) <= REL * l1_scale(imgs[k], T))
    d = decode_peaks(pk)
    assert (int(d["u"][2]), int(d["v"][2])) == (u0, v0)
    with MatchPlan(120, 140, 20, 24, batch=3, write_surface=True, score=N.NCC_SCORE_SAD, shard_rank=1,
                   shard_count=2) as plan:
        _, sb = plan.match(torch.from_numpy(imgs).to(dev), torch.from_numpy(T).to(dev))
        torch.cuda.synchronize()
        a, b = plan.info.u_begin, plan.info.u_end
    np.testing.assert_array_equal(sb.cpu().numpy(), s.cpu().numpy()[:, a:b])


@pytest.mark.parametrize("h,m,step", [(32, 16, 16), (16, 5, 8)])
def test_piv_sad_vectors_and_surfaces(h, m, step):
    p = synth.particle_pair_integer(256, 288, 3, -4, seed=520 + h)
    dev = torch.device("cuda", 0)
    with PivPlan(256, 288, h, m, step, pairs=1, score=N.NCC_SCORE_SAD) as plan:
        assert plan.info.variant_name.decode().startswith("piv_sad")
        vec, sc = plan.correlate(torch.from_numpy(p.A[None].copy()).to(dev), torch.from_numpy(p.B[None].copy()).to(dev),
                                 scores=True)
        torch.cuda.synchronize()
        Ky, Kx = plan.grid
    v = {k: x.cpu().numpy()[0] for k, x in decode_vectors(vec).items()}
    assert np.all(v["iy"] == 3) and np.all(v["ix"] == -4)
    g = synth.rng(521)
    kys, kxs = g.integers(0, Ky, 12), g.integers(0, Kx, 12)
    ref = oracle.piv_windows_sad(p.A, p.B, h, h, m, m, step, step, kys, kxs)
    sc = sc.cpu().numpy()[0]
    for i, (ky, kx) in enumerate(zip(kys, kxs)):
        y, x = m + ky * step, m + kx * step
        A = p.A[y:y + h, x:x + h].astype(np.float64)
        Bw = p.B[y - m:y + h + m, x - m:x + h + m].astype(np.float64)
        E = np.abs(A).sum() + np.abs(Bw).sum()
        assert v["iy"][ky, kx] == ref["iy"][i] and v["ix"][ky, kx] == ref["ix"][i]
        assert v["flags"][ky, kx] == ref["flags"][i]
        assert abs(v["score"][ky, kx] - ref["score"][i]) <= REL * E
        assert abs(v["dy"][ky, kx] - ref["dy"][i]) <= 2e-3 and abs(v["dx"][ky, kx] - ref["dx"][i]) <= 2e-3
        surf = oracle.sad_surface(Bw, A)  # the window's SAD surface = TM SAD of the search region
        assert np.max(np.abs(sc[ky, kx] - surf)) <= REL * E
