"""GPU parity of the persistent warp-specialised PIV kernels at the cfg-4 window shape
(64x64 masks, +-32 search, step 32) and the cfg-3 shape (32x32, +-16, step 16, four windows
per pipeline stage) against the fp64 oracle.

The default kernel (piv_ws2) splits every window's 65x65 offset grid into a 64x64 core
(consumer warps, FFMA2) and a border (last row dy = +32 and last column dx = +32, producer
warps, scalar FFMA + warp sum); the border and the core must agree with the oracle alike, so
the checks include planted peaks on the border and element-wise surfaces.  Each kernel
(piv_ws2, the 13-consumer piv_ws, the non-persistent piv_ncc) is forced in turn through
NCC_FORCE_VARIANT / NCC_NO_WS.  More windows than SMs: the persistent loop runs its two-stage
ring over several windows per CTA.
"""
import numpy as np
import pytest
import torch

import oracle
import synth
from paper_conf_ipps_moorelk13_b200 import _native as N
from paper_conf_ipps_moorelk13_b200 import build as B
from paper_conf_ipps_moorelk13_b200.api import PivPlan, decode_vectors

pytestmark = pytest.mark.gpu
TOL = 1e-4
H, W, h, m, s = 384, 448, 64, 32, 32
# (NCC_PIV_TC=0: these are the CUDA-core kernels; the tensor-core path has test_gpu_piv_tc.py)
KERNELS = {"ws2": ({"NCC_PIV_TC": "0"}, "piv_ws2_64x64_m32_rv16_c8p8"),
           "ws": ({"NCC_PIV_TC": "0", "NCC_FORCE_VARIANT": "piv_ws_64x64_m32_rv12_c13p4"}, "piv_ws_64x64_m32_rv12_c13p4"),
           "ncc": ({"NCC_PIV_TC": "0", "NCC_NO_WS": "1"}, "piv_ws2_64x64_m32_rv16_c8p8")}


@pytest.fixture(scope="module", autouse=True)
def _lib():
    B.build()


def correlate(As, Bs, score=N.NCC_SCORE_NCC, shape=(H, W, h, m, s)):
    dev = torch.device("cuda", 0)
    A = torch.from_numpy(np.ascontiguousarray(np.stack(As))).to(dev)
    Bt = torch.from_numpy(np.ascontiguousarray(np.stack(Bs))).to(dev)
    H_, W_, h_, m_, s_ = shape
    with PivPlan(H_, W_, h_, m_, s_, pairs=len(As), score=score) as plan:
        vec, sc = plan.correlate(A, Bt, scores=True)
        torch.cuda.synchronize()
        info = plan.info.as_dict()
    return {k: v.cpu().numpy() for k, v in decode_vectors(vec).items()}, sc.cpu().numpy(), info


def pairs():
    # shifts on the border of the search range (row +32 / column +32 are the producer's
    # offsets) and inside it; one noisy sub-pixel pair
    out = []
    for i, (dy, dx) in enumerate([(32, -5), (7, 32), (32, 32), (-13, 21)]):
        p = synth.particle_pair_integer(H, W, dy, dx, seed=12000 + i)
        out.append((p.A, p.B, (dy, dx)))
    p = synth.particle_pair_subpixel(H, W, 3.3, -5.6, seed=12010)
    g = synth.rng(12011)
    out.append((p.A + 0.02 * g.standard_normal(p.A.shape).astype(np.float32),
                p.B + 0.02 * g.standard_normal(p.B.shape).astype(np.float32), None))
    return out


@pytest.mark.parametrize("kernel", list(KERNELS))
def test_cfg4_shape_kernels_vs_oracle(kernel, monkeypatch):
    env, name = KERNELS[kernel]
    for k, v in env.items():
        monkeypatch.setenv(k, v)
    ps = pairs()
    v, sc, info = correlate([p[0] for p in ps], [p[1] for p in ps])
    assert info["variant_name"] == name
    Ky, Kx = oracle.piv_grid(H, W, h, h, m, m, s, s)
    assert v["iy"].shape == (len(ps), Ky, Kx) and Ky * Kx * len(ps) > 148
    g = synth.rng(12100)
    for pi, (A, Bf, shift) in enumerate(ps):
        if shift is not None:
            assert np.all(v["iy"][pi] == shift[0]) and np.all(v["ix"][pi] == shift[1])
            assert np.all(np.abs(v["score"][pi] - 1.0) <= TOL)
        kys = np.concatenate([g.integers(0, Ky, 3), [0, Ky - 1]])
        kxs = np.concatenate([g.integers(0, Kx, 3), [Kx - 1, 0]])
        ref = oracle.piv_windows(A, Bf, h, h, m, m, s, s, kys, kxs)
        for i, (ky, kx) in enumerate(zip(kys, kxs)):
            rs = oracle.piv_window_scores(A, Bf, h, h, m, m, s, s, ky, kx)
            d = np.abs(sc[pi, ky, kx] - rs)
            assert d.max() <= TOL, (pi, ky, kx, np.unravel_index(d.argmax(), d.shape))
            assert v["iy"][pi, ky, kx] == ref["iy"][i] and v["ix"][pi, ky, kx] == ref["ix"][i]
            if v["flags"][pi, ky, kx] == ref["flags"][i]:
                assert abs(v["dy"][pi, ky, kx] - ref["dy"][i]) <= 2e-3
                assert abs(v["dx"][pi, ky, kx] - ref["dx"][i]) <= 2e-3
            else:  # a fit branch may flip only on a score within the tolerance of 0
                assert (v["flags"][pi, ky, kx] ^ ref["flags"][i]) & ~np.uint32(8 | 16) == 0


def test_cfg4_shape_ssd_ws2():
    ps = pairs()[:2]
    v, sc, info = correlate([p[0] for p in ps], [p[1] for p in ps], score=N.NCC_SCORE_SSD)
    assert info["variant_name"] == KERNELS["ws2"][1]
    for pi, (A, Bf, shift) in enumerate(ps):
        assert np.all(v["iy"][pi] == shift[0]) and np.all(v["ix"][pi] == shift[1])
        kys, kxs = np.array([0, 3, 7]), np.array([9, 0, 5])
        ref = oracle.piv_windows_ssd(A, Bf, h, h, m, m, s, s, kys, kxs)
        for i, (ky, kx) in enumerate(zip(kys, kxs)):
            Aw = A[m + s * ky:m + s * ky + h, m + s * kx:m + s * kx + h].astype(np.float64)
            E = (Aw ** 2).sum() * 2
            assert abs(v["score"][pi, ky, kx] - ref["score"][i]) <= 1e-5 * E
            assert v["iy"][pi, ky, kx] == ref["iy"][i] and v["ix"][pi, ky, kx] == ref["ix"][i]


KERNELS3 = {"ws2": ({}, "piv_ws2_32x32_m16_rv16_c8p8_w4"),
            "ncc": ({"NCC_NO_WS": "1"}, "piv_ws2_32x32_m16_rv16_c8p8_w4"),
            "sk": ({"NCC_FORCE_VARIANT": "piv_sk_32x32_m16_rv12_nt416_w4"}, "piv_sk_32x32_m16_rv12_nt416_w4")}


@pytest.mark.parametrize("kernel", list(KERNELS3))
def test_cfg3_shape_kernels_vs_oracle(kernel, monkeypatch):
    # 3 pairs x 17 x 19 windows = 969: more 4-window groups than SMs, and a partial last group
    env, name = KERNELS3[kernel]
    for k, v in env.items():
        monkeypatch.setenv(k, v)
    H3, W3, h3, m3, s3 = 320, 352, 32, 16, 16
    ps = []
    for i, (dy, dx) in enumerate([(16, -3), (5, 16), (-16, -16)]):
        p = synth.particle_pair_integer(H3, W3, dy, dx, seed=12200 + i)
        ps.append((p.A, p.B, (dy, dx)))
    v, sc, info = correlate([p[0] for p in ps], [p[1] for p in ps], shape=(H3, W3, h3, m3, s3))
    assert info["variant_name"] == name
    Ky, Kx = oracle.piv_grid(H3, W3, h3, h3, m3, m3, s3, s3)
    assert (Ky, Kx) == (17, 19) and (3 * Ky * Kx) % 4 != 0
    g = synth.rng(12300)
    for pi, (A, Bf, shift) in enumerate(ps):
        assert np.all(v["iy"][pi] == shift[0]) and np.all(v["ix"][pi] == shift[1])
        assert np.all(np.abs(v["score"][pi] - 1.0) <= TOL)
        kys = np.concatenate([g.integers(0, Ky, 4), [0, Ky - 1]])
        kxs = np.concatenate([g.integers(0, Kx, 4), [Kx - 1, 0]])
        ref = oracle.piv_windows(A, Bf, h3, h3, m3, m3, s3, s3, kys, kxs)
        for i, (ky, kx) in enumerate(zip(kys, kxs)):
            rs = oracle.piv_window_scores(A, Bf, h3, h3, m3, m3, s3, s3, ky, kx)
            d = np.abs(sc[pi, ky, kx] - rs)
            assert d.max() <= TOL, (pi, ky, kx, np.unravel_index(d.argmax(), d.shape))
            assert v["flags"][pi, ky, kx] == ref["flags"][i]
            assert abs(v["dy"][pi, ky, kx] - ref["dy"][i]) <= 2e-3
            assert abs(v["dx"][pi, ky, kx] - ref["dx"][i]) <= 2e-3
