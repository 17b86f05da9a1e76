"""GPU parity: the tensor-core PIV numerator (piv_tc_kernel, tcgen05 kind::f16 3xBF16, R image
rows per MMA) through the C ABI vs the fp64 oracle.

Same bar as the CUDA-core PIV tests: window score surfaces within 1e-4 element by
element, integer displacements bit-exact on planted shifts, flags equal, sub-pixel |d delta| <= 2e-3
where both sides took the same fit branch.  Plus: the strip segmentation (which windows share a
CTA's Hankel operand) does not change any result bit.
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


@pytest.fixture(autouse=True)
def _force_tc(monkeypatch):
    """The tensor-core kernel for every eligible geometry (by default only the +-32 search, where
    it is the faster one, takes it)."""
    monkeypatch.setenv("NCC_PIV_TC", "1")


def run(As, Bs, h, search, step, scores=True):
    As = np.ascontiguousarray(np.stack(As))
    Bs = np.ascontiguousarray(np.stack(Bs))
    P, H, W = As.shape
    dev = torch.device("cuda", 0)
    with PivPlan(H, W, h, search, step, pairs=P) as plan:
        vec, sc = plan.correlate(torch.from_numpy(As).to(dev), torch.from_numpy(Bs).to(dev), scores=scores)
        torch.cuda.synchronize()
        info = plan.info.as_dict()
        out = {k: v.cpu().numpy() for k, v in decode_vectors(vec).items()}
        return out, (sc.cpu().numpy() if sc is not None else None), info


def _hw(x):
    return (x, x) if np.isscalar(x) else tuple(x)


def check_windows(A, Bf, v, sc, pi, h, w, my, mx, sy, sx, kys, kxs):
    ref = oracle.piv_windows(A, Bf, h, w, my, mx, sy, sx, kys, kxs)
    for i, (ky, kx) in enumerate(zip(kys, kxs)):
        rs = oracle.piv_window_scores(A, Bf, h, w, my, mx, sy, sx, ky, kx)
        err = np.max(np.abs(sc[pi, ky, kx] - rs))
        assert err <= TOL, (pi, ky, kx, err)
        assert v["flags"][pi, ky, kx] == ref["flags"][i]
        assert v["iy"][pi, ky, kx] == ref["iy"][i] and v["ix"][pi, ky, kx] == ref["ix"][i]
        assert abs(v["dy"][pi, ky, kx] - ref["dy"][i]) <= 2e-3
        assert abs(v["dx"][pi, ky, kx] - ref["dx"][i]) <= 2e-3


def test_cfg3_planted_all_windows_on_tensor_cores():
    c = synth.CONFIGS[3]
    dy, dx = synth.piv_shift_for_pair(3, 0)
    p = synth.particle_pair_integer(c["H"], c["W"], dy, dx, seed=3000)
    v, sc, info = run([p.A], [p.B], 32, 16, 16)
    assert info["variant_name"].startswith("piv_tc_bf16x3_32x32_m16x16_r4"), info["variant_name"]
    assert info["specialized"] == 3
    assert np.all(v["iy"] == dy) and np.all(v["ix"] == dx)
    assert np.all(np.abs(v["score"] - 1.0) <= TOL)
    g = synth.rng(3002)
    kys = np.concatenate([g.integers(0, 61, 24), [0, 60, 0, 60, 30]])
    kxs = np.concatenate([g.integers(0, 61, 24), [0, 60, 60, 0, 30]])
    check_windows(p.A, p.B, v, sc, 0, 32, 32, 16, 16, 16, 16, kys, kxs)


def test_cfg4_geometry_all_windows_two_pairs():
    """64^2 masks, +-32, step 32 (cfg 4's window geometry, R = 2) on 384^2 crops of two
    canvases: every window's whole 65 x 65 surface against the oracle."""
    cv, specs = synth.piv_batch_from_canvases(4, 2, canvases=2)
    As, Bs = [], []
    for (ci, ay, ax, by, bx, _) in specs:
        As.append(cv[ci][ay:ay + 384, ax:ax + 384])
        Bs.append(cv[ci][by:by + 384, bx:bx + 384])
    v, sc, info = run(As, Bs, 64, 32, 32)
    assert info["variant_name"].startswith("piv_tc_bf16x3_64x64_m32x32_r2"), info["variant_name"]
    Ky, Kx = oracle.piv_grid(384, 384, 64, 64, 32, 32, 32, 32)
    assert v["iy"].shape == (2, Ky, Kx)
    for pi, (_, _, _, _, _, (dy, dx)) in enumerate(specs):
        assert np.all(v["iy"][pi] == dy) and np.all(v["ix"][pi] == dx)
        kk = np.array([(a, b) for a in range(Ky) for b in range(Kx)])
        check_windows(As[pi], Bs[pi], v, sc, pi, 64, 64, 32, 32, 32, 32, kk[:, 0], kk[:, 1])


def test_cfg4_full_frames_sampled():
    cv, specs = synth.piv_batch_from_canvases(4, 2, canvases=2)
    As, Bs = [], []
    for (ci, ay, ax, by, bx, _) in specs:
        As.append(cv[ci][ay:ay + 2048, ax:ax + 2048])
        Bs.append(cv[ci][by:by + 2048, bx:bx + 2048])
    v, sc, info = run(As, Bs, 64, 32, 32)
    assert info["specialized"] == 3
    for pi, (_, _, _, _, _, (dy, dx)) in enumerate(specs):
        assert np.all(v["iy"][pi] == dy) and np.all(v["ix"][pi] == dx)
        g = synth.rng(4100 + pi)
        kys = np.concatenate([g.integers(0, 61, 5), [0, 60]])
        kxs = np.concatenate([g.integers(0, 61, 5), [60, 0]])
        check_windows(As[pi], Bs[pi], v, sc, pi, 64, 64, 32, 32, 32, 32, kys, kxs)


def test_noisy_subpixel_pair_vs_oracle():
    p = synth.particle_pair_subpixel(512, 512, -7.3, 4.6, seed=3200)
    g = synth.rng(3201)
    A = p.A + 0.02 * g.standard_normal(p.A.shape).astype(np.float32)
    Bn = p.B + 0.02 * g.standard_normal(p.B.shape).astype(np.float32)
    v, sc, info = run([A], [Bn], 32, 16, 16)
    assert info["specialized"] == 3
    Ky, Kx = v["iy"].shape[1:]
    kys, kxs = g.integers(0, Ky, 40), g.integers(0, Kx, 40)
    ref = oracle.piv_windows(A, Bn, 32, 32, 16, 16, 16, 16, kys, kxs)
    gv = {k: v[k][0, kys, kxs] for k in v}
    assert np.all(gv["iy"] == ref["iy"]) and np.all(gv["ix"] == ref["ix"])
    assert np.all(np.abs(gv["score"] - ref["score"]) <= TOL)
    same = gv["flags"] == ref["flags"]
    assert same.mean() > 0.9
    assert np.abs(gv["dy"] - ref["dy"])[same].max() <= 2e-3
    assert np.abs(gv["dx"] - ref["dx"])[same].max() <= 2e-3


@pytest.mark.parametrize("h,w,my,mx,sy,sx", [
    (48, 32, 16, 16, 24, 16),  # rectangular mask, step 24 (4 live windows per strip row)
    (32, 16, 8, 16, 12, 8),    # m_y != m_x
    (64, 48, 32, 32, 32, 20),  # 48 template columns (3 chunks), odd window count per row
    (16, 64, 4, 32, 8, 4),     # D_x = 64 with a short mask and a tight step
])
def test_other_geometries(h, w, my, mx, sy, sx):
    H, W = 200 + 2 * my, 240 + 2 * mx
    p = synth.particle_pair_integer(H, W, 3, -2, seed=5100 + h + w)
    v, sc, info = run([p.A], [p.B], (h, w), (my, mx), (sy, sx))
    assert info["specialized"] == 3, info["variant_name"]
    Ky, Kx = oracle.piv_grid(H, W, h, w, my, mx, sy, sx)
    ref = oracle.piv_pair(p.A, p.B, h, w, my, mx, sy, sx)
    np.testing.assert_array_equal(v["iy"][0], ref["iy"])
    np.testing.assert_array_equal(v["ix"][0], ref["ix"])
    np.testing.assert_array_equal(v["flags"][0], ref["flags"])
    assert np.max(np.abs(v["score"][0] - ref["score"])) <= TOL
    for ky, kx in [(0, 0), (Ky - 1, Kx - 1), (Ky // 2, Kx // 3), (Ky - 1, 0)]:
        rs = oracle.piv_window_scores(p.A, p.B, h, w, my, mx, sy, sx, ky, kx)
        assert np.max(np.abs(sc[0, ky, kx] - rs)) <= TOL


def test_flat_masks_and_zero_shift():
    p = synth.particle_pair_integer(256, 256, 0, 0, seed=6100)
    A = p.A.copy()
    A[0:64, 0:64] = 0.0
    v, _, info = run([A], [p.B], 32, 16, 16, scores=False)
    assert info["specialized"] == 3
    ref = oracle.piv_pair(A, p.B, 32, 32, 16, 16, 16, 16)
    np.testing.assert_array_equal(v["flags"][0], ref["flags"])
    assert v["flags"][0, 0, 0] & 32
    ok = (ref["flags"] & 32) == 0
    assert np.all(v["iy"][0][ok] == 0) and np.all(v["ix"][0][ok] == 0)


@pytest.mark.parametrize("segw", ["1", "3", "7"])
def test_strip_segmentation_bitwise(segw, monkeypatch):
    """Which windows share a CTA's Hankel operand (strip segments) changes no bit: every window's
    accumulation sequence is fixed by its own geometry.  Sub-batches of one pair as well."""
    cv, specs = synth.piv_batch_from_canvases(4, 3, canvases=2)
    As = np.stack([cv[ci][ay:ay + 512, ax:ax + 512] for (ci, ay, ax, by, bx, _) in specs])
    Bs = np.stack([cv[ci][by:by + 512, bx:bx + 512] for (ci, ay, ax, by, bx, _) in specs])
    v0, s0, _ = run(list(As), list(Bs), 64, 32, 32)
    monkeypatch.setenv("NCC_PIV_TC_SEGW", segw)
    monkeypatch.setenv("NCC_PIV_SUB_BATCH", "1")
    v1, s1, _ = run(list(As), list(Bs), 64, 32, 32)
    np.testing.assert_array_equal(s0, s1)
    for k in v0:
        np.testing.assert_array_equal(v0[k], v1[k])


def test_cuda_core_kernel_still_selectable(monkeypatch):
    monkeypatch.setenv("NCC_PIV_TC", "0")
    p = synth.particle_pair_integer(512, 512, 4, -6, seed=3300)
    v, sc, info = run([p.A], [p.B], 32, 16, 16)
    assert info["variant_name"].startswith("piv_ws2"), info["variant_name"]
    assert np.all(v["iy"] == 4) and np.all(v["ix"] == -6)


def test_default_selection(monkeypatch):
    """Without NCC_PIV_TC the plan takes the tensor cores at +-32 (R = 2, where they measured
    faster) and the CUDA-core kernel at +-16."""
    monkeypatch.delenv("NCC_PIV_TC", raising=False)
    with PivPlan(512, 512, 64, 32, 32, pairs=1) as plan:
        assert plan.info.variant_name.decode().startswith("piv_tc_bf16x3_64x64_m32x32_r2")
    with PivPlan(512, 512, 32, 16, 16, pairs=1) as plan:
        assert plan.info.variant_name.decode().startswith("piv_ws2")


def test_equal_sub_batches_and_host_chunks_bitwise(monkeypatch):
    """The tensor-core path's sub-batching (equal-sized sub-batches within an 8 GiB factors budget;
    NCC_PIV_SUB_BATCH caps it) and the host path's streamed chunks change no bit: 5 pairs as one
    launch, as sub-batches of 2 + 2 + 1, and through piv_correlate_host in chunks."""
    cv, specs = synth.piv_batch_from_canvases(4, 5, canvases=2)
    As = np.ascontiguousarray(np.stack([cv[ci][ay:ay + 384, ax:ax + 384] for (ci, ay, ax, by, bx, _) in specs]))
    Bs = np.ascontiguousarray(np.stack([cv[ci][by:by + 384, bx:bx + 384] for (ci, ay, ax, by, bx, _) in specs]))
    v0, s0, info = run(list(As), list(Bs), 64, 32, 32)
    assert info["variant_name"].startswith("piv_tc"), info["variant_name"]
    monkeypatch.setenv("NCC_PIV_SUB_BATCH", "2")
    v1, s1, _ = run(list(As), list(Bs), 64, 32, 32)
    np.testing.assert_array_equal(s0, s1)
    for k in v0:
        np.testing.assert_array_equal(v0[k], v1[k])
    hA = torch.from_numpy(As).pin_memory()
    hB = torch.from_numpy(Bs).pin_memory()
    with PivPlan(384, 384, 64, 32, 32, pairs=5) as plan:
        hv = torch.full((5,) + plan.grid + (6,), -1, dtype=torch.int32).pin_memory()
        for _ in range(2):  # the second call reuses the chunk slots
            plan.correlate_host(hA, hB, hv)
        torch.cuda.synchronize()
    d = {k: x.numpy() for k, x in decode_vectors(hv).items()}
    for k in v0:
        np.testing.assert_array_equal(d[k], v0[k])
    for pi, (_, _, _, _, _, (dy, dx)) in enumerate(specs):
        assert np.all(v0["iy"][pi] == dy) and np.all(v0["ix"][pi] == dx)
