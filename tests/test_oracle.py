"""Pins for the fp64 CPU oracle (no GPU).

The oracle (oracle/ncc_oracle.c) is checked against things other than itself:
  * hand-derived closed forms (tests/golden/hand_cases.json),
  * numpy.corrcoef (library Pearson) on random non-square cases,
  * invariants the corr2 definition fixes (planted = 1, |r| <= 1, affine invariance,
    symmetry, flat -> 0),
  * an independent algebra (oracle/ncc_fft.py: FFT numerator + fp64 SAT denominator),
  * PIV: planted integer shifts, the window-grid count by enumeration, sub-pixel closed
    forms (Gaussian / parabola triples are recovered exactly), the SSD minimum fit
    (exact parabolas, mirrored triples, a fractional-shift particle pair), and the flat
    threshold (templates straddling 1e-10 of the raw energy).
Citations: PAPER.md Fig 5.1 caption P:132-137 (definition), Listing 5.1 caption
P:250-251 (corr2 per shift), PIV Figs 5.9-5.12 captions P:165-171; SURVEY.md 8(c).
"""
import json
import math
import os

import numpy as np
import pytest

import oracle
from oracle.ncc_fft import ncc_surface_fft, window_sums
import synth

GOLD = os.path.join(os.path.dirname(__file__), "golden", "hand_cases.json")


def _closed(expr: str) -> float:
    return float(eval(expr, {"sqrt": math.sqrt}))


def _cases():
    with open(GOLD) as f:
        return json.load(f)


# ---------------------------------------------------------------- hand cases
def test_hand_case_A():
    c = _cases()["case_A"]
    s = oracle.ncc_surface(np.array(c["image"], np.float32), np.array(c["template"], np.float32))
    exp = np.array([[_closed(e) for e in row] for row in c["expected"]])
    np.testing.assert_allclose(s, exp, rtol=0, atol=1e-14)


def test_hand_case_B():
    c = _cases()["case_B"]
    s = oracle.ncc_surface(np.array(c["image"], np.float32), np.array(c["template"], np.float32))
    for u, v, e in c["expected_at"]:
        assert abs(s[u, v] - _closed(e)) < 1e-14, (u, v, s[u, v], e)
    # negated image -> -1 at the plant (alpha < 0 flips the sign)
    s2 = oracle.ncc_surface(-np.array(c["image"], np.float32), np.array(c["template"], np.float32))
    assert abs(s2[1, 1] + 1.0) < 1e-14


def test_hand_case_E_flat():
    c = _cases()["case_E_flat"]
    s = oracle.ncc_surface(np.array(c["image"], np.float32), np.array(c["template"], np.float32))
    exp = np.array([[_closed(e) for e in row] for row in c["expected"]])
    np.testing.assert_allclose(s, exp, rtol=0, atol=1e-14)


# ---------------------------------------------------------------- library routine
@pytest.mark.parametrize("H,W,h,w,seed", [(9, 11, 3, 5, 1), (12, 7, 4, 2, 2), (10, 10, 7, 3, 3), (6, 13, 1, 6, 4)])
def test_matches_numpy_corrcoef(H, W, h, w, seed):
    g = synth.rng(seed)
    I = g.random((H, W), dtype=np.float32)
    T = g.random((h, w), dtype=np.float32) * 3 - 1
    s = oracle.ncc_surface(I, T)
    assert s.shape == (H - h + 1, W - w + 1)
    for u in range(H - h + 1):
        for v in range(W - w + 1):
            ref = np.corrcoef(T.astype(np.float64).ravel(), I[u:u + h, v:v + w].astype(np.float64).ravel())[0, 1]
            assert abs(s[u, v] - ref) < 1e-12


def test_ncc_at_matches_surface():
    I, T, _, _ = synth.tm_inputs(1)
    s = oracle.ncc_surface(I, T)
    g = synth.rng(5)
    us = g.integers(0, s.shape[0], 50)
    vs = g.integers(0, s.shape[1], 50)
    np.testing.assert_array_equal(oracle.ncc_at(I, T, us, vs), s[us, vs])


def test_band_rows():
    I, T, _, _ = synth.tm_inputs(1)
    s = oracle.ncc_surface(I, T)
    np.testing.assert_array_equal(oracle.ncc_surface(I, T, 10, 23), s[10:23])


# ---------------------------------------------------------------- invariants
def test_planted_scores_one_and_is_peak():
    I, T, u0, v0 = synth.tm_inputs(1)
    s, pk = oracle.ncc_match(I, T)
    assert abs(s[u0, v0] - 1.0) < 1e-12
    assert (pk.u, pk.v) == (u0, v0) and pk.valid
    assert np.all(np.abs(s) <= 1.0 + 1e-12)


def test_affine_invariance():
    g = synth.rng(11)
    I = g.random((20, 23), dtype=np.float32)
    T = g.random((5, 7), dtype=np.float32)
    s = oracle.ncc_surface(I, T)
    np.testing.assert_allclose(oracle.ncc_surface(2.5 * I - 7, T), s, atol=1e-6)  # fp32 input rounding
    np.testing.assert_allclose(oracle.ncc_surface(I, 0.25 * T + 3), s, atol=1e-6)
    np.testing.assert_allclose(oracle.ncc_surface(-I, T), -s, atol=1e-12)
    np.testing.assert_allclose(oracle.ncc_surface(I, -T), -s, atol=1e-12)
    # exactly representable affine maps (power-of-two scale, small shift) -> tight agreement
    Iq = synth.quantize(I)
    sq = oracle.ncc_surface(Iq, T)
    np.testing.assert_allclose(oracle.ncc_surface(4 * Iq + 1, T), sq, atol=1e-13)


def test_symmetry_template_window():
    g = synth.rng(12)
    A = g.random((6, 9), dtype=np.float32)
    B = g.random((6, 9), dtype=np.float32)
    assert abs(oracle.ncc_surface(A, B)[0, 0] - oracle.ncc_surface(B, A)[0, 0]) < 1e-15


def test_flat_template_all_zero_and_invalid():
    I = synth.uniform_image(16, 16, 3)
    T = np.full((4, 4), 0.3, np.float32)
    s, pk = oracle.ncc_match(I, T)
    assert np.all(s == 0.0) and not pk.valid and (pk.u, pk.v) == (0, 0)


def test_flat_window_zero():
    I = synth.uniform_image(16, 16, 4)
    I[2:8, 3:9] = 0.75
    T = synth.uniform_image(4, 4, 5)
    s = oracle.ncc_surface(I, T)
    assert np.all(s[2:5, 3:6] == 0.0)
    assert np.all(s[6:, :] != 0.0)


def test_argmax_tie_smallest_index():
    s = np.zeros((5, 7))
    s[3, 1] = s[1, 4] = s[4, 6] = 0.9
    assert oracle.argmax(s) == 1 * 7 + 4


# ---------------------------------------------------------------- independent algebra
@pytest.mark.parametrize("smooth", [False, True])
def test_bruteforce_equals_fft_route(smooth):
    img = synth.smooth_image(96, 80, 21) if smooth else synth.uniform_image(96, 80, 21)
    T, _, _ = synth.planted_template(img, 17, 13, 22)
    s = oracle.ncc_surface(img, T)
    f = ncc_surface_fft(img, T)
    assert np.max(np.abs(s - f)) < 1e-10


def test_window_sums_exact_on_quantized():
    img = synth.quantize(synth.uniform_image(40, 33, 7))
    S1, S2 = window_sums(img, 9, 5)
    I = img.astype(np.float64)
    for u in (0, 5, 31):
        for v in (0, 11, 28):
            assert S1[u, v] == I[u:u + 9, v:v + 5].sum()
            assert S2[u, v] == (I[u:u + 9, v:v + 5] ** 2).sum()


# ---------------------------------------------------------------- PIV
def test_piv_grid_by_enumeration():
    for (H, W, h, w, my, mx, sy, sx) in [(1024, 1024, 32, 32, 16, 16, 16, 16), (2048, 2048, 64, 64, 32, 32, 32, 32),
                                         (100, 77, 8, 6, 3, 2, 5, 4)]:
        ny = len([y for y in range(my, H, sy) if y + h + my <= H])
        nx = len([x for x in range(mx, W, sx) if x + w + mx <= W])
        assert oracle.piv_grid(H, W, h, w, my, mx, sy, sx) == (ny, nx)
    assert oracle.piv_grid(1024, 1024, 32, 32, 16, 16, 16, 16) == (61, 61)
    assert oracle.piv_grid(2048, 2048, 64, 64, 32, 32, 32, 32) == (61, 61)


def test_piv_planted_integer_shift():
    dy, dx = 3, -5
    p = synth.particle_pair_integer(160, 176, dy, dx, seed=31)
    v = oracle.piv_pair(p.A, p.B, 32, 32, 8, 8, 16, 16)
    assert np.all(v["iy"] == dy) and np.all(v["ix"] == dx)
    assert np.all(np.abs(v["score"] - 1.0) < 1e-9)
    assert np.all(v["flags"] & (oracle.EDGE_Y | oracle.EDGE_X | oracle.INVALID) == 0)
    # Integer-shift peaks have symmetric-ish neighbours; the fit stays inside (-0.5, 0.5)
    assert np.all(np.abs(v["dy"] - dy) < 0.5) and np.all(np.abs(v["dx"] - dx) < 0.5)


def test_piv_zero_shift():
    p = synth.particle_pair_integer(96, 96, 0, 0, seed=32)
    v = oracle.piv_pair(p.A, p.A, 16, 16, 4, 4, 16, 16)
    assert np.all(v["iy"] == 0) and np.all(v["ix"] == 0)
    assert np.all(np.abs(v["score"] - 1.0) < 1e-12)


def test_piv_scores_are_tm_surface_of_search_region():
    p = synth.particle_pair_integer(128, 128, 2, 1, seed=33)
    h = w = 16
    m = 6
    s = 16
    ky, kx = 2, 3
    y, x = m + ky * s, m + kx * s
    sc = oracle.piv_window_scores(p.A, p.B, h, w, m, m, s, s, ky, kx)
    ref = oracle.ncc_surface(p.B[y - m:y + h + m, x - m:x + w + m], p.A[y:y + h, x:x + w])
    np.testing.assert_array_equal(sc, ref)


def test_piv_edge_flags():
    # true shift beyond the search radius -> peak can land on the border
    p = synth.particle_pair_integer(128, 128, 9, 0, seed=34)
    v = oracle.piv_pair(p.A, p.B, 16, 16, 4, 4, 16, 16)
    on_edge = np.abs(v["iy"]) == 4
    assert on_edge.any()
    assert np.all((v["flags"][on_edge] & oracle.EDGE_Y) != 0)
    assert np.all(v["dy"][on_edge] == v["iy"][on_edge])


def test_piv_flat_mask_invalid():
    A = np.zeros((64, 64), np.float32)
    B = synth.uniform_image(64, 64, 35)
    v = oracle.piv_pair(A, B, 16, 16, 4, 4, 16, 16)
    assert np.all(v["flags"] & oracle.INVALID) and np.all(v["score"] == 0.0)


# ---------------------------------------------------------------- sub-pixel
def test_subpixel_symmetric_is_zero():
    assert oracle.subpixel3(0.5, 0.9, 0.5) == (0.0, False)
    assert oracle.subpixel3(-0.2, 0.9, -0.2) == (0.0, True)


@pytest.mark.parametrize("delta,sigma", [(0.3, 1.0), (-0.17, 0.8), (0.45, 1.6), (-0.49, 1.2)])
def test_subpixel_gaussian_exact(delta, sigma):
    c = [math.exp(-((k - delta) ** 2) / (2 * sigma * sigma)) for k in (-1, 0, 1)]
    d, par = oracle.subpixel3(*c)
    assert not par and abs(d - delta) < 1e-12


@pytest.mark.parametrize("delta", [0.21, -0.33, 0.05])
def test_subpixel_parabola_fallback_exact(delta):
    a, b = 0.3, 0.5
    c = [a - b * (k - delta) ** 2 for k in (-1, 0, 1)]
    assert min(c) <= 0  # forces the parabolic branch
    d, par = oracle.subpixel3(*c)
    assert par and abs(d - delta) < 1e-12


def test_subpixel_not_a_maximum():
    assert oracle.subpixel3(0.9, 0.5, 0.9)[0] == 0.0
    assert oracle.subpixel3(0.5, 0.5, 0.5)[0] == 0.0


def test_piv_subpixel_recovers_fractional_shift():
    p = synth.particle_pair_subpixel(160, 160, 2.3, -1.6, seed=36)
    v = oracle.piv_pair(p.A, p.B, 32, 32, 6, 6, 16, 16)
    assert np.all(v["iy"] == 2) and np.all(v["ix"] == -2)
    # method accuracy (reported, not a parity bound): Gaussian fit within 0.1 px here
    assert np.median(np.abs(v["dy"] - 2.3)) < 0.1
    assert np.median(np.abs(v["dx"] + 1.6)) < 0.1


# ---------------------------------------------------------------- SSD (paper's PIV metric, Fig 5.10)
def test_ssd_hand_case():
    # case A windows are [[a,a+1],[a+3,a+4]] (a = 1,2,4,5) vs T = [[1,2],[3,4]]:
    # T - W = [[1-a, 1-a], [-a, -a]] -> SSD = 2(1-a)^2 + 2a^2 = 2, 10, 50, 82
    c = _cases()["case_A"]
    s = oracle.ssd_surface(np.array(c["image"], np.float32), np.array(c["template"], np.float32))
    np.testing.assert_array_equal(s, np.array([[2.0, 10.0], [50.0, 82.0]]))


def test_ssd_invariants():
    img, T, u0, v0 = synth.tm_inputs(1)
    s, pk = oracle.ssd_match(img, T)
    assert s[u0, v0] == 0.0 and (pk.u, pk.v) == (u0, v0)
    assert np.all(s >= 0.0)
    # symmetry and the expansion sum T^2 - 2 sum T W + sum W^2 through an independent path
    g = synth.rng(44)
    A = g.random((5, 7), dtype=np.float32)
    B = g.random((5, 7), dtype=np.float32)
    assert oracle.ssd_surface(A, B)[0, 0] == oracle.ssd_surface(B, A)[0, 0]
    a, b = A.astype(np.float64), B.astype(np.float64)
    assert abs(oracle.ssd_surface(A, B)[0, 0] - ((a * a).sum() - 2 * (a * b).sum() + (b * b).sum())) < 1e-12
    # shift invariance: adding c to both template and image leaves SSD unchanged
    sq = oracle.ssd_surface(synth.quantize(img), synth.quantize(T))
    np.testing.assert_allclose(oracle.ssd_surface(synth.quantize(img) + 2, synth.quantize(T) + 2), sq, atol=1e-9)


def test_argmin_tie_smallest_index():
    s = np.ones((4, 6))
    s[2, 1] = s[0, 5] = s[3, 3] = 0.1
    assert oracle.argmin(s) == 5


def test_piv_ssd_planted_shift_and_parabola():
    p = synth.particle_pair_integer(160, 176, -2, 4, seed=45)
    v = oracle.piv_windows_ssd(p.A, p.B, 32, 32, 8, 8, 16, 16, [1, 2, 3], [1, 4, 2])
    assert np.all(v["iy"] == -2) and np.all(v["ix"] == 4) and np.all(v["score"] < 1e-9)


# ---------------------------------------------------------------- SSD sub-pixel (Fig 5.10: argmin + parabola)
@pytest.mark.parametrize("delta,a,b", [(0.3, 1.0, 2.0), (-0.2, 0.0, 0.5), (0.49, 7.5, 0.01), (-0.45, 3.0, 40.0)])
def test_subpixel3_min_exact_parabola(delta, a, b):
    """Closed form: c_k = a + b (k - delta)^2 (b > 0) is a parabola with its minimum at delta;
    the oracle's 3-point minimum fit must return delta exactly (to rounding)."""
    c = [a + b * (k - delta) ** 2 for k in (-1, 0, 1)]
    assert abs(oracle.subpixel3_min(*c) - delta) < 1e-12


def test_subpixel3_min_special_cases():
    assert oracle.subpixel3_min(2.0, 1.0, 2.0) == 0.0     # symmetric -> 0
    assert oracle.subpixel3_min(1.0, 2.0, 1.0) == 0.0     # a maximum, not a minimum -> no fit
    assert oracle.subpixel3_min(1.0, 1.0, 1.0) == 0.0     # flat -> no fit
    # sign: the lower neighbour pulls the vertex towards it
    assert oracle.subpixel3_min(1.0, 0.5, 2.0) < 0.0 < oracle.subpixel3_min(2.0, 0.5, 1.0)
    # the maximum fit (NCC) and the minimum fit (SSD) agree on mirrored triples: delta of
    # (c-, c0, c+) as a minimum == delta of (-c-, -c0, -c+) as a maximum (parabolic branch)
    for tri in [(3.0, 1.0, 2.0), (5.0, 0.2, 0.9)]:
        d_min = oracle.subpixel3_min(*tri)
        d_max, par = oracle.subpixel3(*[-x for x in tri])
        assert par and abs(d_min - d_max) < 1e-15


def test_piv_ssd_fractional_shift_sign_and_magnitude():
    """SSD PIV on a particle pair re-rendered at a known fractional shift (2.3, -1.6): the
    integer argmin is the nearest integer shift and the oracle's parabolic sub-pixel estimate
    moves towards the planted value with the right sign on both axes (bias of the 3-point
    parabola on 2.6-px particles is well under 0.25 px)."""
    p = synth.particle_pair_subpixel(160, 160, 2.3, -1.6, seed=37)
    v = oracle.piv_windows_ssd(p.A, p.B, 32, 32, 6, 6, 16, 16, [1, 2, 3, 4, 2], [1, 3, 2, 4, 4])
    assert np.all(v["iy"] == 2) and np.all(v["ix"] == -2)
    assert np.all(v["flags"] & (oracle.EDGE_Y | oracle.EDGE_X) == 0)
    fy, fx = v["dy"] - v["iy"], v["dx"] - v["ix"]
    assert np.all(fy > 0) and np.all(fx > 0)  # 2 -> 2.3 (up), -2 -> -1.6 (up)
    assert np.median(np.abs(v["dy"] - 2.3)) < 0.25 and np.median(np.abs(v["dx"] + 1.6)) < 0.25


# ---------------------------------------------------------------- flat threshold (S8c reading 4)
def _checker(n: int, base: float, delta: float) -> np.ndarray:
    s = np.where((np.add.outer(np.arange(n), np.arange(n)) % 2) == 0, 1.0, -1.0)
    return (base + delta * s).astype(np.float32)


def test_flat_threshold_relative_to_raw_energy():
    """Flat <=> sum (T - Tbar)^2 <= 1e-10 * sum T^2.  A 4x4 checkerboard 4 +- d has centred
    energy 16 d^2 and raw energy ~256, ratio d^2 / 16 (all values exact in fp32):
      d = 2^-15: ratio 5.8e-11 -> flat;  d = 2^-13: ratio 9.3e-10 -> not flat.
    The d = 2^-15 case is NOT flat under an absolute threshold (16 d^2 = 1.5e-8 > 1e-10) nor
    under a threshold based on sum T (1e-10 * 64 = 6.4e-9 < 1.5e-8), so either mistake fails.
    Tiny-valued templates (2^-20 scale, centred energy ~1e-13) are flat under an absolute
    threshold but not under the relative one.  Scaling by a power of two never changes it."""
    assert oracle.template_is_flat(_checker(4, 4.0, 2.0 ** -15))
    assert not oracle.template_is_flat(_checker(4, 4.0, 2.0 ** -13))
    for k in (-6, 0, 10):
        assert oracle.template_is_flat(_checker(4, 4.0, 2.0 ** -15) * np.float32(2.0 ** k))
        assert not oracle.template_is_flat(_checker(4, 4.0, 2.0 ** -13) * np.float32(2.0 ** k))
    tiny = (synth.uniform_image(6, 5, 38) * np.float32(2.0 ** -20)).astype(np.float32)
    assert not oracle.template_is_flat(tiny)
    # and corr2 returns 0 for the flat one / a finite score for the other
    img = synth.uniform_image(12, 12, 39)
    assert np.all(oracle.ncc_surface(img, _checker(4, 4.0, 2.0 ** -15)) == 0.0)
    assert np.all(oracle.ncc_surface(img, _checker(4, 4.0, 2.0 ** -13)) != 0.0)


# ---------------------------------------------------------------- SAD (Ch. 4 specialisation example)
def test_sad_hand_case():
    # case A windows are [[a,a+1],[a+3,a+4]] (a = 1,2,4,5) vs T = [[1,2],[3,4]]:
    # T - W = [[1-a, 1-a], [-a, -a]] -> SAD = 2|1-a| + 2|a| = 2, 6, 14, 18
    c = _cases()["case_A"]
    s = oracle.sad_surface(np.array(c["image"], np.float32), np.array(c["template"], np.float32))
    np.testing.assert_array_equal(s, np.array([[2.0, 6.0], [14.0, 18.0]]))


def test_sad_invariants_and_bounds():
    """SAD >= 0, = 0 at the plant, symmetric, invariant to a common shift, and bounded by the
    SSD through Cauchy-Schwarz: SSD / max|T - W| <= SAD <= sqrt(n * SSD) (n = h w)."""
    img, T, u0, v0 = synth.tm_inputs(1)
    s, pk = oracle.sad_match(img, T)
    assert s[u0, v0] == 0.0 and (pk.u, pk.v) == (u0, v0)
    assert np.all(s >= 0.0)
    g = synth.rng(46)
    A = g.random((5, 7), dtype=np.float32)
    B = g.random((5, 7), dtype=np.float32)
    assert oracle.sad_surface(A, B)[0, 0] == oracle.sad_surface(B, A)[0, 0]
    q = synth.quantize(img)
    tq = synth.quantize(T)
    np.testing.assert_array_equal(oracle.sad_surface(q + 2, tq + 2), oracle.sad_surface(q, tq))
    sad = oracle.sad_surface(img, T)
    ssd = oracle.ssd_surface(img, T)
    n = T.size
    assert np.all(sad <= np.sqrt(n * ssd) * (1 + 1e-12) + 1e-12)
    d = np.abs(T.astype(np.float64) - img[3:19, 5:21].astype(np.float64))
    assert ssd[3, 5] / d.max() <= sad[3, 5] * (1 + 1e-12)


def test_piv_sad_planted_shift():
    p = synth.particle_pair_integer(160, 176, 3, -4, seed=47)
    v = oracle.piv_windows_sad(p.A, p.B, 32, 32, 8, 8, 16, 16, [1, 2, 3], [1, 4, 2])
    assert np.all(v["iy"] == 3) and np.all(v["ix"] == -4) and np.all(v["score"] == 0.0)
    # the sub-pixel step is the same minimum fit as SSD's (pinned above): at an exact integer
    # shift the SAD surface is V-shaped around 0, the parabola's vertex stays within (-0.5, 0.5)
    assert np.all(np.abs(v["dy"] - 3) < 0.5) and np.all(np.abs(v["dx"] + 4) < 0.5)
