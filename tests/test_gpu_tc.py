"""GPU parity of the tensor-core numerator (tcgen05 kind::f16 with the
3xBF16 split, ncc_tc.cuh) through the C ABI vs the fp64 oracle: full surfaces within 1e-4,
planted peaks exact, SSD, several template blocks (h > 128, w > 128), batches, band shards
bitwise equal to the full problem (the per-output accumulation order does not depend on the
band), and the CUDA-core path agreeing within the tolerance."""
import numpy as np
import pytest
import torch

import oracle
import synth
from oracle.ncc_fft import ncc_surface_fft
from paper_conf_ipps_moorelk13_b200 import _native as N
from paper_conf_ipps_moorelk13_b200 import build as B
from paper_conf_ipps_moorelk13_b200.api import MatchPlan, decode_peaks
from _peaks import assert_peak_ok

pytestmark = pytest.mark.gpu
TOL = 1e-4


@pytest.fixture(scope="module", autouse=True)
def _lib():
    B.build()


@pytest.fixture(autouse=True)
def _tc(monkeypatch):
    monkeypatch.setenv("NCC_TC", "1")  # tensor cores whenever eligible (the default picks by cost)


def test_tc_is_default_for_cfg2_and_not_for_small_templates(monkeypatch):
    monkeypatch.delenv("NCC_TC")
    with MatchPlan(1024, 1024, 128, 128) as plan:
        assert plan.info.variant_name.decode().startswith("tm_tc")
    with MatchPlan(1024, 1024, 128, 128, cuda_cores=True) as plan:
        assert not plan.info.variant_name.decode().startswith("tm_tc")
    with MatchPlan(64, 64, 16, 16) as plan:
        assert not plan.info.variant_name.decode().startswith("tm_tc")


def run(imgs, T, shard=(0, 1), score=N.NCC_SCORE_NCC):
    imgs = np.ascontiguousarray(np.stack(imgs))
    F, H, W = imgs.shape
    h, w = T.shape
    dev = torch.device("cuda", 0)
    with MatchPlan(H, W, h, w, batch=F, write_surface=True, shard_rank=shard[0], shard_count=shard[1],
                   score=score) as plan:
        pk, s = plan.match(torch.from_numpy(imgs).to(dev), torch.from_numpy(np.ascontiguousarray(T)).to(dev))
        torch.cuda.synchronize()
        info = plan.info.as_dict()
    return {k: v.cpu().numpy() for k, v in decode_peaks(pk).items()}, s.cpu().numpy(), info


@pytest.mark.parametrize("H,W,h,w", [(64, 64, 16, 16), (300, 420, 37, 300), (400, 380, 200, 150),
                                     (260, 200, 129, 33), (150, 700, 8, 8)])
def test_tc_shapes_vs_oracle(H, W, h, w):
    img = synth.uniform_image(H, W, h + w)
    T, u0, v0 = synth.planted_template(img, h, w, 3 * h)
    ref, pk = oracle.ncc_match(img, T)
    peaks, s, info = run([img], T)
    assert info["variant_name"].startswith("tm_tc"), info["variant_name"]
    assert np.max(np.abs(s[0] - ref)) <= TOL
    assert (peaks["u"][0], peaks["v"][0]) == (u0, v0) == (pk.u, pk.v)


@pytest.mark.parametrize("smooth", [False, True])
def test_tc_cfg2_full_surface(smooth):
    img, T, u0, v0 = synth.tm_inputs(2, smooth=smooth)
    peaks, s, info = run([img], T)
    assert info["variant_name"].startswith("tm_tc"), info["variant_name"]
    f = ncc_surface_fft(img, T)
    assert np.max(np.abs(s[0] - f)) <= TOL
    g = synth.rng(97)
    us, vs = g.integers(0, 897, 200), g.integers(0, 897, 200)
    assert np.max(np.abs(s[0][us, vs] - oracle.ncc_at(img, T, us, vs))) <= TOL
    assert (peaks["u"][0], peaks["v"][0]) == (u0, v0)


def test_tc_bands_bitwise_and_batch():
    imgs = [synth.uniform_image(330, 290, 60 + k) for k in range(2)]
    T, _, _ = synth.planted_template(imgs[1], 40, 36, 61)
    full_pk, full, _ = run(imgs, T)
    parts = [run(imgs, T, shard=(r, 3))[1] for r in range(3)]
    np.testing.assert_array_equal(np.concatenate(parts, axis=1), full)
    for k in range(2):
        ref, pk = oracle.ncc_match(imgs[k], T)
        assert np.max(np.abs(full[k] - ref)) <= TOL
        if k == 1:  # planted: exact
            assert (full_pk["u"][k], full_pk["v"][k]) == (pk.u, pk.v)
        else:  # no planted match: SURVEY 8(c) reading 5 (near-tie rule)
            assert_peak_ok(int(full_pk["u"][k]), int(full_pk["v"][k]), ref)


def test_tc_ssd():
    img = synth.uniform_image(200, 260, 71)
    T, u0, v0 = synth.planted_template(img, 30, 50, 72)
    ref = oracle.ssd_surface(img, T)
    peaks, s, _ = run([img], T, score=N.NCC_SCORE_SSD)
    assert np.max(np.abs(s[0] - ref)) <= 1e-5 * float(2 * (T.astype(np.float64) ** 2).sum() + 10)
    assert (peaks["u"][0], peaks["v"][0]) == (u0, v0)


def test_tc_matches_cuda_core_path(monkeypatch):
    img, T, u0, v0 = synth.tm_inputs(2, k=4)
    _, s_tc, _ = run([img], T)
    monkeypatch.setenv("NCC_TC", "0")
    _, s_cc, info = run([img], T)
    assert not info["variant_name"].startswith("tm_tc")
    assert np.max(np.abs(s_tc - s_cc)) <= TOL


def test_tc_unaligned_pitch_falls_back_at_run_time():
    """pitch % 4 != 0: the image split (tm_tc_split) reads rows with scalar loads; the
    tensor-core kernel reads its own (hi, lo) copy through TMA; results stay exact."""
    img, T, u0, v0 = synth.tm_inputs(2, k=9)
    H, W = img.shape
    P = W + 1
    buf = np.zeros((H, P), np.float32)
    buf[:, :W] = img
    dev = torch.device("cuda", 0)
    with MatchPlan(H, W, 128, 128, write_surface=True, image_pitch=P) as plan:
        assert plan.info.variant_name.decode().startswith("tm_tc")
        pk, s = plan.match(torch.from_numpy(buf).to(dev), torch.from_numpy(T).to(dev))
        torch.cuda.synchronize()
    d = decode_peaks(pk)
    assert (int(d["u"][0]), int(d["v"][0])) == (u0, v0)
    g = synth.rng(96)
    us, vs = g.integers(0, 897, 100), g.integers(0, 897, 100)
    assert np.max(np.abs(s[0].cpu().numpy()[us, vs] - oracle.ncc_at(img, T, us, vs))) <= TOL


def test_tc_host_path_matches_device_path():
    img, T, u0, v0 = synth.tm_inputs(2, k=11)
    peaks, s, _ = run([img], T)
    hp = torch.empty((1, 4), dtype=torch.int32).pin_memory()
    with MatchPlan(1024, 1024, 128, 128) as plan:
        assert plan.info.variant_name.decode().startswith("tm_tc")
        plan.match_host(torch.from_numpy(img[None].copy()).pin_memory(), torch.from_numpy(T).pin_memory(), hp)
        torch.cuda.synchronize()
    d = decode_peaks(hp)
    assert (int(d["u"][0]), int(d["v"][0])) == (peaks["u"][0], peaks["v"][0]) == (u0, v0)
    assert float(d["score"][0]) == float(peaks["score"][0])


@pytest.mark.parametrize("h,w", [(128, 128), (129, 129), (32, 32), (128, 33), (255, 64)])
def test_tc_block_boundaries(h, w):
    """Template sizes at and just past the 128-row block and 32-column chunk boundaries."""
    img = synth.uniform_image(h + 170, w + 150, 3 * h + w)
    T, u0, v0 = synth.planted_template(img, h, w, 7 * h + w)
    ref, pk = oracle.ncc_match(img, T)
    peaks, s, info = run([img], T)
    assert info["variant_name"].startswith("tm_tc")
    assert np.max(np.abs(s[0] - ref)) <= TOL
    assert (peaks["u"][0], peaks["v"][0]) == (u0, v0)


@pytest.mark.parametrize("H,W,h,w", [(400, 556, 300, 300), (380, 555, 260, 299)])
def test_tc_large_template_ragged_columns(H, W, h, w):
    """Templates wider than 256 with a ragged last output column (V = 1 mod 128): the ragged
    column comes from tm_tc_cols_rw (4 sliding output rows per warp) and the window sums from the
    two-pass form; full surface vs the fp64 oracle, planted peak exact.  W = 555: the staged
    (hi, lo) rows are padded to an even number of pairs (16-byte TMA stride)."""
    img = synth.uniform_image(H, W, h + w + 1)
    T, u0, v0 = synth.planted_template(img, h, w, 3 * h + 1)
    ref, pk = oracle.ncc_match(img, T)
    peaks, s, info = run([img], T)
    assert info["variant_name"].startswith("tm_tc") and info["variant_name"].endswith("_cols"), info["variant_name"]
    assert np.max(np.abs(s[0] - ref)) <= TOL
    assert np.max(np.abs(s[0][:, -2:] - ref[:, -2:])) <= TOL
    assert (int(peaks["u"][0]), int(peaks["v"][0])) == (pk.u, pk.v) == (u0, v0)


@pytest.mark.parametrize("smooth", [False, True])
def test_tc_cfg5_full_surface_fft(smooth, monkeypatch):
    """cfg5 (4096^2 frame, 512^2 template) on the DEFAULT tensor-core plan, uniform and the
    smooth cancellation-stress variant (App. A.3's worst fp32 case): full surface
    vs the independent fp64 FFT route (pinned to brute force in test_oracle.py), brute-force
    samples including the ragged last column, planted peak exact."""
    monkeypatch.delenv("NCC_TC")  # the default plan, not the forced one
    img, T, u0, v0 = synth.tm_inputs(5, k=3, smooth=smooth)
    peaks, s, info = run([img], T)
    assert info["variant_name"].startswith("tm_tc"), info["variant_name"]
    f = ncc_surface_fft(img, T)
    assert np.max(np.abs(s[0] - f)) <= TOL
    g = synth.rng(99)
    us = np.concatenate([g.integers(0, 3585, 24), [u0, 3584, 0, 1792]])
    vs = np.concatenate([g.integers(0, 3585, 24), [v0, 3584, 3584, 3584]])
    bf = oracle.ncc_at(img, T, us, vs)
    assert np.max(np.abs(s[0][us, vs] - bf)) <= TOL
    assert (int(peaks["u"][0]), int(peaks["v"][0])) == (u0, v0)


@pytest.mark.parametrize("pinned", [True, False])
def test_tc_host_path_surface_after_a_different_frame(monkeypatch, pinned):
    """on the tensor-core plan the host path's frame copy must be ordered
    before every kernel that reads the frame, including the ragged-column kernel on the side
    stream (V % 128 == 1 at cfg2).  Alternate two frames through ncc_match_host and compare the
    WHOLE surface, bit for bit, with the device path on the same frame."""
    monkeypatch.delenv("NCC_TC")
    frames = [synth.tm_inputs(2, k=30 + k) for k in range(2)]
    T = frames[0][1]
    dev = torch.device("cuda", 0)
    ref = []
    with MatchPlan(1024, 1024, 128, 128, write_surface=True) as plan:
        assert plan.info.variant_name.decode().endswith("_cols")
        for img, _, _, _ in frames:
            pk, s = plan.match(torch.from_numpy(img).to(dev), torch.from_numpy(T).to(dev))
            ref.append((s[0].cpu().numpy(), pk.cpu().numpy()))
        hT = torch.from_numpy(T)
        hp = torch.empty((1, 4), dtype=torch.int32)
        hs = torch.empty((1, 897, 897), dtype=torch.float32)
        himgs = [torch.from_numpy(f[0][None].copy()) for f in frames]
        if pinned:
            hT, hp, hs = hT.pin_memory(), hp.pin_memory(), hs.pin_memory()
            himgs = [h.pin_memory() for h in himgs]
        for it in range(4):
            k = it % 2
            plan.match_host(himgs[k], hT, hp, h_scores=hs)
            torch.cuda.synchronize()
            np.testing.assert_array_equal(hs[0].numpy(), ref[k][0])
            np.testing.assert_array_equal(hp.numpy(), ref[k][1])
    assert (int(ref[0][1][0, 1]), int(ref[0][1][0, 2])) == (frames[0][2], frames[0][3])
