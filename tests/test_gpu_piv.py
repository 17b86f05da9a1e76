"""GPU parity: PIV batched correlation + peak + sub-pixel through the C ABI vs the oracle.

Bar: window score surfaces within 1e-4 of the fp64 oracle element by element; integer
displacements bit-exact on planted-shift particle pairs; sub-pixel |d delta| <= 2e-3 px
where both sides took the same fit branch and the peak curvature is <= -0.05
(SURVEY 8(c) pins); flags equal.
"""
import numpy as np
import pytest
import torch

import oracle
import synth
from paper_conf_ipps_moorelk13_b200 import build as B
from paper_conf_ipps_moorelk13_b200.api import PivPlan, decode_vectors

pytestmark = pytest.mark.gpu
TOL = 1e-4


@pytest.fixture(scope="module", autouse=True)
def _lib():
    B.build()


def run_piv(As, Bs, h, m, s, generic=False, scores=True, search=None, step=None):
    As = np.ascontiguousarray(np.stack(As))
    Bs = np.ascontiguousarray(np.stack(Bs))
    P, H, W = As.shape
    dev = torch.device("cuda", 0)
    with PivPlan(H, W, h, m if search is None else search, s if step is None else step, pairs=P,
                 generic=generic) as plan:
        vec, sc = plan.correlate(torch.from_numpy(As).to(dev), torch.from_numpy(Bs).to(dev), scores=scores)
        torch.cuda.synchronize()
        info = plan.info.as_dict()
        out = {k: v.cpu().numpy() for k, v in decode_vectors(vec).items()}
        return out, (sc.cpu().numpy() if sc is not None else None), info


def check_subpixel(gpu, ref_vecs, mask=None):
    same = (gpu["flags"] == ref_vecs["flags"])
    if mask is not None:
        same &= mask
    d = np.abs(gpu["dy"] - ref_vecs["dy"])[same]
    e = np.abs(gpu["dx"] - ref_vecs["dx"])[same]
    return same, d, e


def test_cfg3_planted_integer_shift_all_windows():
    c = synth.CONFIGS[3]
    dy, dx = synth.piv_shift_for_pair(3, 0)
    p = synth.particle_pair_integer(c["H"], c["W"], dy, dx, seed=3000)
    v, sc, info = run_piv([p.A], [p.B], 32, 16, 16)
    assert info["specialized"] == 1 and (info["Ky"], info["Kx"]) == (61, 61)
    assert np.all(v["iy"] == dy) and np.all(v["ix"] == dx)
    assert np.all(np.abs(v["score"] - 1.0) <= TOL)
    # element-wise score surfaces + full vector records on sampled windows
    g = synth.rng(3001)
    kys = np.concatenate([g.integers(0, 61, 40), [0, 60, 0, 60]])
    kxs = np.concatenate([g.integers(0, 61, 40), [0, 60, 60, 0]])
    ref = oracle.piv_windows(p.A, p.B, 32, 32, 16, 16, 16, 16, kys, kxs)
    for i, (ky, kx) in enumerate(zip(kys, kxs)):
        rs = oracle.piv_window_scores(p.A, p.B, 32, 32, 16, 16, 16, 16, ky, kx)
        assert np.max(np.abs(sc[0, ky, kx] - rs)) <= TOL
        assert v["iy"][0, ky, kx] == ref["iy"][i] and v["ix"][0, ky, kx] == ref["ix"][i]
        assert v["flags"][0, ky, kx] == ref["flags"][i]
        assert abs(v["dy"][0, ky, kx] - ref["dy"][i]) <= 2e-3
        assert abs(v["dx"][0, ky, kx] - ref["dx"][i]) <= 2e-3


def test_cfg3_noisy_subpixel_pair_vs_oracle():
    p = synth.particle_pair_subpixel(1024, 1024, 3.3, -5.6, seed=3100)
    g = synth.rng(3101)
    A = p.A + 0.02 * g.standard_normal(p.A.shape).astype(np.float32)
    Bn = p.B + 0.02 * g.standard_normal(p.B.shape).astype(np.float32)
    v, sc, _ = run_piv([A], [Bn], 32, 16, 16)
    kys = g.integers(0, 61, 60)
    kxs = g.integers(0, 61, 60)
    ref = oracle.piv_windows(A, Bn, 32, 32, 16, 16, 16, 16, kys, kxs)
    gv = {k: v[k][0, kys, kxs] for k in v}
    assert np.all(gv["iy"] == ref["iy"]) and np.all(gv["ix"] == ref["ix"])
    assert np.all(np.abs(gv["score"] - ref["score"]) <= TOL)
    same, d, e = check_subpixel(gv, ref)
    assert same.mean() > 0.9
    assert d.max() <= 2e-3 and e.max() <= 2e-3


def test_cfg4_two_pairs_sampled(monkeypatch):
    monkeypatch.setenv("NCC_PIV_TC", "0")  # the CUDA-core kernel (tensor cores: test_gpu_piv_tc.py)
    cv, specs = synth.piv_batch_from_canvases(4, 2, canvases=2)
    As, Bs = [], []
    for (ci, ay, ax, by, bx, _) in specs:
        As.append(cv[ci][ay:ay + 2048, ax:ax + 2048])
        Bs.append(cv[ci][by:by + 2048, bx:bx + 2048])
    v, sc, info = run_piv(As, Bs, 64, 32, 32, scores=True)
    assert info["specialized"] == 1
    for pi, (_, _, _, _, _, (dy, dx)) in enumerate(specs):
        assert np.all(v["iy"][pi] == dy) and np.all(v["ix"][pi] == dx)
        g = synth.rng(4000 + pi)
        kys, kxs = g.integers(0, 61, 6), g.integers(0, 61, 6)
        ref = oracle.piv_windows(As[pi], Bs[pi], 64, 64, 32, 32, 32, 32, kys, kxs)
        for i, (ky, kx) in enumerate(zip(kys, kxs)):
            rs = oracle.piv_window_scores(As[pi], Bs[pi], 64, 64, 32, 32, 32, 32, ky, kx)
            assert np.max(np.abs(sc[pi, ky, kx] - rs)) <= TOL
            assert v["flags"][pi, ky, kx] == ref["flags"][i]
            assert v["iy"][pi, ky, kx] == ref["iy"][i] and v["ix"][pi, ky, kx] == ref["ix"][i]
            assert abs(v["dy"][pi, ky, kx] - ref["dy"][i]) <= 2e-3
            assert abs(v["dx"][pi, ky, kx] - ref["dx"][i]) <= 2e-3


@pytest.mark.parametrize("h,w,my,mx,sy,sx", [(24, 20, 5, 7, 9, 11), (16, 16, 4, 4, 8, 8), (32, 32, 16, 16, 16, 16),
                                             (13, 29, 3, 0, 7, 5)])
@pytest.mark.parametrize("generic", [True, False])
@pytest.mark.parametrize("W", [170, 168])  # 170: plain loads (pitch); 168: TMA when step_x % 4 == 0
def test_odd_shapes_generic_and_runtime_specialised(h, w, my, mx, sy, sx, generic, W):
    p = synth.particle_pair_integer(150, W, 2, -3, seed=5000 + h)
    v, sc, info = run_piv([p.A], [p.B], (h, w), None, None, generic=generic, search=(my, mx), step=(sy, sx))
    aot = (h, w, my, mx) == (32, 32, 16, 16)
    assert info["specialized"] == (0 if generic else (1 if aot else 2)), info["variant_name"]
    Ky, Kx = oracle.piv_grid(150, W, h, w, my, mx, sy, sx)
    assert v["iy"].shape == (1, Ky, Kx)
    ref = oracle.piv_pair(p.A, p.B, h, w, my, mx, sy, sx)
    np.testing.assert_array_equal(v["iy"][0], ref["iy"])
    np.testing.assert_array_equal(v["ix"][0], ref["ix"])
    np.testing.assert_array_equal(v["flags"][0], ref["flags"])
    assert np.max(np.abs(v["score"][0] - ref["score"])) <= TOL
    for ky, kx in [(0, 0), (Ky - 1, Kx - 1), (Ky // 2, Kx // 3)]:
        rs = oracle.piv_window_scores(p.A, p.B, h, w, my, mx, sy, sx, ky, kx)
        assert np.max(np.abs(sc[0, ky, kx] - rs)) <= TOL


def test_zero_shift_and_flat_mask():
    p = synth.particle_pair_integer(256, 256, 0, 0, seed=6000)
    A = p.A.copy()
    A[0:64, 0:64] = 0.0  # flat masks in the top-left windows
    v, _, _ = run_piv([A], [p.B], 32, 16, 16, scores=False)
    ref = oracle.piv_pair(A, p.B, 32, 32, 16, 16, 16, 16)
    np.testing.assert_array_equal(v["flags"][0], ref["flags"])
    assert v["flags"][0, 0, 0] & 32
    ok = (ref["flags"] & 32) == 0
    assert np.all(v["iy"][0][ok] == 0) and np.all(v["ix"][0][ok] == 0)


def test_host_path_matches_device_path():
    p = synth.particle_pair_integer(512, 512, -4, 6, seed=7000)
    v, _, _ = run_piv([p.A], [p.B], 32, 16, 16, scores=False)
    hA = torch.from_numpy(p.A[None].copy()).pin_memory()
    hB = torch.from_numpy(p.B[None].copy()).pin_memory()
    with PivPlan(512, 512, 32, 16, 16, pairs=1) as plan:
        hv = torch.empty((1,) + plan.grid + (6,), dtype=torch.int32).pin_memory()
        plan.correlate_host(hA, hB, hv)
        torch.cuda.synchronize()
    d = decode_vectors(hv)
    np.testing.assert_array_equal(d["iy"].numpy(), v["iy"])
    np.testing.assert_array_equal(d["dy"].numpy(), v["dy"])


@pytest.mark.parametrize("sub_batch", [1, 2])
def test_host_path_streams_chunks(monkeypatch, sub_batch):
    """Host path with more pairs than one sub-batch: chunks stream through two device slots
    (copy of chunk c+1 overlapping the correlation of chunk c); vectors equal the device path."""
    P = 5
    pairs = [synth.particle_pair_integer(256, 256, 3 - k, k - 2, seed=7100 + k) for k in range(P)]
    v, _, _ = run_piv([p.A for p in pairs], [p.B for p in pairs], 32, 16, 16, scores=False)
    monkeypatch.setenv("NCC_PIV_SUB_BATCH", str(sub_batch))
    hA = torch.from_numpy(np.stack([p.A for p in pairs])).pin_memory()
    hB = torch.from_numpy(np.stack([p.B for p in pairs])).pin_memory()
    with PivPlan(256, 256, 32, 16, 16, pairs=P) as plan:
        hv = torch.full((P,) + plan.grid + (6,), -1, dtype=torch.int32).pin_memory()
        for _ in range(2):  # the second call reuses the slots after the first call's chunks
            plan.correlate_host(hA, hB, hv)
        torch.cuda.synchronize()
    d = decode_vectors(hv)
    for k in ("iy", "ix", "dy", "dx", "score", "flags"):
        np.testing.assert_array_equal(d[k].numpy(), v[k])
    for k in range(P):
        assert (d["iy"][k] == 3 - k).all() and (d["ix"][k] == k - 2).all()


def test_unaligned_pitch_plain_loads():
    p = synth.particle_pair_integer(256, 256, 5, 2, seed=8000)
    P = 259
    A = np.zeros((1, 256, P), np.float32)
    B_ = np.zeros((1, 256, P), np.float32)
    A[0, :, :256] = p.A
    B_[0, :, :256] = p.B
    dev = torch.device("cuda", 0)
    with PivPlan(256, 256, 32, 16, 16, pairs=1, image_pitch=P) as plan:
        vec, sc = plan.correlate(torch.from_numpy(A).to(dev), torch.from_numpy(B_).to(dev), scores=True)
        torch.cuda.synchronize()
        assert plan.info.specialized == 1
    d = {k: v.cpu().numpy() for k, v in decode_vectors(vec).items()}
    ref = oracle.piv_pair(p.A, p.B, 32, 32, 16, 16, 16, 16)
    np.testing.assert_array_equal(d["iy"][0], ref["iy"])
    np.testing.assert_array_equal(d["ix"][0], ref["ix"])
    rs = oracle.piv_window_scores(p.A, p.B, 32, 32, 16, 16, 16, 16, 5, 6)
    assert np.max(np.abs(sc[0, 5, 6].cpu().numpy() - rs)) <= TOL


def test_partial_last_window_group():
    # Ky*Kx not a multiple of the windows-per-CTA of the specialised cfg3 kernel
    p = synth.particle_pair_integer(32 * 7 + 32, 32 * 5 + 32, -3, 4, seed=8100)
    H, W = p.A.shape
    v, sc, info = run_piv([p.A], [p.B], 32, 16, 16)
    Ky, Kx = oracle.piv_grid(H, W, 32, 32, 16, 16, 16, 16)
    assert (Ky * Kx) % 4 != 0
    assert np.all(v["iy"][0] == -3) and np.all(v["ix"][0] == 4)
