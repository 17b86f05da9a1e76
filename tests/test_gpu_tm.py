"""GPU parity: template matching (TM) through the C ABI vs the fp64 oracle.

Bar (BASELINE.json north_star): max |dNCC| <= 1e-4 element by element; peak locations
bit-exact on planted inputs.  Sizes: the oracle full surface where it finishes in seconds
(several tiles + ragged tails), and at full BASELINE sizes the independent FFT route
(itself pinned to the brute force in test_oracle.py) plus brute-force samples.
"""
import numpy as np
import pytest
import torch

import oracle
from oracle.ncc_fft import ncc_surface_fft
import synth
from paper_conf_ipps_moorelk13_b200 import build as B
from paper_conf_ipps_moorelk13_b200 import shard
from paper_conf_ipps_moorelk13_b200.api import MatchPlan, decode_peaks
from _peaks import assert_peak_ok

pytestmark = pytest.mark.gpu
TOL = 1e-4


@pytest.fixture(scope="module", autouse=True)
def _lib():
    B.build()


def run_match(img, T, generic=False, batch_imgs=None, shard=(0, 1)):
    imgs = np.stack(batch_imgs) if batch_imgs is not None else img[None]
    H, W = imgs.shape[1:]
    h, w = T.shape
    dev = torch.device("cuda", 0)
    with MatchPlan(H, W, h, w, batch=imgs.shape[0], write_surface=True, generic=generic,
                   shard_rank=shard[0], shard_count=shard[1], cuda_cores=True) as plan:
        d_img = torch.from_numpy(imgs).to(dev)
        d_t = torch.from_numpy(np.ascontiguousarray(T)).to(dev)
        peaks, scores = plan.match(d_img, d_t)
        torch.cuda.synchronize()
        info = plan.info.as_dict()
        return {k: v.cpu().numpy() for k, v in decode_peaks(peaks).items()}, scores.cpu().numpy(), info


@pytest.mark.parametrize("generic", [False, True])
def test_cfg1_full_surface(generic):
    img, T, u0, v0 = synth.tm_inputs(1)
    ref, pk = oracle.ncc_match(img, T)
    peaks, s, info = run_match(img, T, generic)
    assert info["specialized"] == (0 if generic else 1)
    assert np.max(np.abs(s[0] - ref)) <= TOL
    assert (peaks["u"][0], peaks["v"][0]) == (u0, v0) == (pk.u, pk.v)
    assert peaks["flags"][0] == 0
    assert abs(peaks["score"][0] - 1.0) <= TOL


@pytest.mark.parametrize("smooth", [False, True])
def test_cfg1_default_plan_full_surface(smooth):
    """cfg1 (64^2 / 16^2) on the DEFAULT plan (the one-launch tm_tiny_kernel), uniform and the
    smooth cancellation-stress variant of SURVEY 8(d): full surface vs the fp64 oracle, planted
    peak exact."""
    img, T, u0, v0 = synth.tm_inputs(1, smooth=smooth)
    ref, pk = oracle.ncc_match(img, T)
    dev = torch.device("cuda", 0)
    with MatchPlan(64, 64, 16, 16, write_surface=True) as plan:
        assert plan.info.variant_name.decode().startswith("tm_tiny"), plan.info.variant_name
        peaks, s = plan.match(torch.from_numpy(img).to(dev), torch.from_numpy(T).to(dev))
        torch.cuda.synchronize()
    d = decode_peaks(peaks)
    assert np.max(np.abs(s[0].cpu().numpy() - ref)) <= TOL
    assert (int(d["u"][0]), int(d["v"][0])) == (u0, v0) == (pk.u, pk.v)


@pytest.mark.parametrize("base,delta,flat", [(4.0, 2.0 ** -15, True), (4.0, 2.0 ** -13, False)])
@pytest.mark.parametrize("cuda_cores", [True, False])
def test_flat_threshold_straddle(base, delta, flat, cuda_cores, monkeypatch):
    """SURVEY 8(c) reading 4 on the GPU: checkerboard templates whose centred / raw energy ratio
    straddles 1e-10 (pinned in test_oracle.py::test_flat_threshold_relative_to_raw_energy) get
    the oracle's flat decision -- FLAT_TEMPLATE|INVALID and an all-zero surface for the flat one,
    a valid peak and oracle-equal scores for the other (CUDA-core and tensor-core templates)."""
    h = w = 4 if cuda_cores else 144
    if not cuda_cores:
        monkeypatch.setenv("NCC_TC", "1")  # tensor cores whenever eligible (small problem)
    sgn = np.where((np.add.outer(np.arange(h), np.arange(w)) % 2) == 0, 1.0, -1.0)
    T = (base + delta * sgn).astype(np.float32)
    assert oracle.template_is_flat(T) == flat
    img = synth.uniform_image(h + 60, w + 70, 41)
    dev = torch.device("cuda", 0)
    with MatchPlan(h + 60, w + 70, h, w, write_surface=True, cuda_cores=cuda_cores) as plan:
        if not cuda_cores:
            assert plan.info.variant_name.decode().startswith("tm_tc"), plan.info.variant_name
        peaks, s = plan.match(torch.from_numpy(img).to(dev), torch.from_numpy(T).to(dev))
        torch.cuda.synchronize()
    d = decode_peaks(peaks)
    s = s[0].cpu().numpy()
    if flat:
        assert int(d["flags"][0]) & 1 and int(d["flags"][0]) & 32
        assert np.all(s == 0.0)
    else:
        assert int(d["flags"][0]) == 0
        ref = oracle.ncc_surface(img, T)
        assert np.max(np.abs(s - ref)) <= TOL


@pytest.mark.parametrize("H,W,h,w,smooth", [(100, 137, 23, 17, False), (157, 123, 33, 41, True),
                                            (300, 280, 156, 116, False), (70, 90, 1, 1, False),
                                            (64, 64, 64, 64, False), (41, 300, 7, 290, False)])
@pytest.mark.parametrize("generic", [True, False])
def test_ragged_shapes_generic_and_runtime_specialised(H, W, h, w, smooth, generic):
    """generic=True: run-time-evaluated kernel; False: NVRTC-specialised for (h, w)."""
    img = synth.smooth_image(H, W, 7) if smooth else synth.uniform_image(H, W, 7)
    T, u0, v0 = synth.planted_template(img, h, w, 8)
    ref, pk = oracle.ncc_match(img, T)
    peaks, s, info = run_match(img, T, generic=generic)
    assert info["specialized"] == (0 if generic else 2), info["variant_name"]
    assert np.max(np.abs(s[0] - ref)) <= TOL
    if h * w > 1:
        assert (peaks["u"][0], peaks["v"][0]) == (u0, v0)


@pytest.mark.parametrize("smooth", [False, True])
def test_cfg2_full_surface_fft_and_samples(smooth):
    img, T, u0, v0 = synth.tm_inputs(2, smooth=smooth)
    peaks, s, info = run_match(img, T)
    assert info["specialized"] == 1
    f = ncc_surface_fft(img, T)
    assert np.max(np.abs(s[0] - f)) <= TOL
    g = synth.rng(99)
    us = np.concatenate([g.integers(0, 897, 300), np.arange(u0 - 2, u0 + 3).repeat(5), [0, 896, 896]])
    vs = np.concatenate([g.integers(0, 897, 300), np.tile(np.arange(v0 - 2, v0 + 3), 5), [896, 0, 896]])
    ok = (us >= 0) & (us < 897) & (vs >= 0) & (vs < 897)
    us, vs = us[ok], vs[ok]
    bf = oracle.ncc_at(img, T, us, vs)
    assert np.max(np.abs(s[0][us, vs] - bf)) <= TOL
    assert (peaks["u"][0], peaks["v"][0]) == (u0, v0)


def test_cfg2_rows_vs_bruteforce_band():
    img, T, u0, v0 = synth.tm_inputs(2, k=1)
    peaks, s, _ = run_match(img, T)
    ref = oracle.ncc_surface(img, T, 0, 40)  # full rows, all columns, including the ragged tail
    assert np.max(np.abs(s[0][:40] - ref)) <= TOL


@pytest.mark.slow
def test_cfg5_full_surface_fft_and_samples():
    img, T, u0, v0 = synth.tm_inputs(5)
    peaks, s, info = run_match(img, T)
    assert info["specialized"] == 1
    f = ncc_surface_fft(img, T)
    assert np.max(np.abs(s[0] - f)) <= TOL
    g = synth.rng(98)
    us = np.concatenate([g.integers(0, 3585, 48), [u0, u0 - 1, u0 + 1, 3584, 0]])
    vs = np.concatenate([g.integers(0, 3585, 48), [v0, v0 + 1, v0 - 1, 3584, 3584]])
    bf = oracle.ncc_at(img, T, us, vs)
    assert np.max(np.abs(s[0][us, vs] - bf)) <= TOL
    assert (peaks["u"][0], peaks["v"][0]) == (u0, v0)


def test_batch_frames_and_host_path():
    imgs = [synth.uniform_image(200, 180, 40 + k) for k in range(3)]
    T, _, _ = synth.planted_template(imgs[1], 24, 20, 3)
    peaks, s, _ = run_match(None, T, batch_imgs=imgs)
    for k in range(3):
        ref, pk = oracle.ncc_match(imgs[k], T)
        assert np.max(np.abs(s[k] - ref)) <= TOL
        if k == 1:  # planted: exact
            assert (peaks["u"][k], peaks["v"][k]) == (pk.u, pk.v)
        else:  # no planted match: SURVEY 8(c) reading 5 (near-tie rule)
            assert_peak_ok(int(peaks["u"][k]), int(peaks["v"][k]), ref)
    # host-buffer entry point gives the same peaks
    stack = torch.from_numpy(np.stack(imgs)).pin_memory()
    tt = torch.from_numpy(T).pin_memory()
    hp = torch.empty((3, 4), dtype=torch.int32).pin_memory()
    with MatchPlan(200, 180, 24, 20, batch=3, cuda_cores=True) as plan:
        plan.match_host(stack, tt, hp)
        torch.cuda.synchronize()
    d = decode_peaks(hp)
    np.testing.assert_array_equal(d["u"].numpy(), peaks["u"])
    np.testing.assert_array_equal(d["v"].numpy(), peaks["v"])
    np.testing.assert_array_equal(d["score"].numpy(), peaks["score"])


def test_band_shards_cover_and_merge():
    img, T, u0, v0 = synth.tm_inputs(1, k=3)
    full_peaks, full, _ = run_match(img, T)
    parts, keys = [], []
    for r in range(3):
        pk, s, info = run_match(img, T, shard=(r, 3))
        assert s.shape[1] == info["u_end"] - info["u_begin"]
        assert (info["u_begin"], info["u_end"]) == shard.band_range(49, r, 3)
        parts.append(s[0])
        keys.append((pk["score"][0], -(pk["u"][0] * 49 + pk["v"][0]), pk["u"][0], pk["v"][0]))
    np.testing.assert_array_equal(np.concatenate(parts, axis=0), full[0])  # bitwise: order independent of band
    best = max(keys)
    assert (best[2], best[3]) == (full_peaks["u"][0], full_peaks["v"][0]) == (u0, v0)


def test_flat_template_and_flat_windows():
    img = synth.uniform_image(80, 90, 50)
    img[10:40, 20:60] = 0.25
    T = synth.uniform_image(8, 8, 51)
    peaks, s, _ = run_match(img, T)
    ref = oracle.ncc_surface(img, T)
    assert np.max(np.abs(s[0] - ref)) <= TOL
    assert np.all(s[0][10:33, 20:53] == 0.0)
    Tf = np.full((8, 8), 0.5, np.float32)
    peaks, s, _ = run_match(img, Tf)
    assert np.all(s[0] == 0.0)
    assert peaks["flags"][0] & 1 and peaks["flags"][0] & 32
    assert (peaks["u"][0], peaks["v"][0]) == (0, 0)


def test_tie_break_smallest_index():
    # periodic image: the template matches exactly at several offsets -> smallest u*V+v
    tile = synth.quantize(synth.uniform_image(8, 8, 60))  # exact window sums -> bitwise-equal ties
    img = np.tile(tile, (6, 6))
    T = np.ascontiguousarray(img[8:16, 8:16])
    peaks, s, _ = run_match(img, T)
    ones = np.argwhere(s[0] >= 1.0 - 1e-6)
    assert len(ones) > 1
    assert (peaks["u"][0], peaks["v"][0]) == tuple(ones[0])


def test_timing_and_info():
    img, T, _, _ = synth.tm_inputs(2)
    dev = torch.device("cuda", 0)
    with MatchPlan(1024, 1024, 128, 128, timing=True) as plan:
        d_img = torch.from_numpy(img).to(dev)
        d_t = torch.from_numpy(T).to(dev)
        plan.match(d_img, d_t)
        t = plan.timing()
        assert t.numerator_ms > 0 and t.total_ms >= t.numerator_ms and t.numerator_launches == 1
        assert plan.info.regs_per_thread > 0
        assert abs(plan.info.flops_per_call - 2 * 128 * 128 * 897 * 897) < 1


def test_unaligned_pitch_uses_plain_loads():
    """pitch % 4 != 0 -> no TMA (plain-load kernel); same numbers as the oracle."""
    img, T, u0, v0 = synth.tm_inputs(1, k=7)
    H, W = img.shape
    P = W + 3
    buf = np.zeros((H, P), np.float32)
    buf[:, :W] = img
    dev = torch.device("cuda", 0)
    with MatchPlan(H, W, 16, 16, write_surface=True, image_pitch=P, cuda_cores=True) as plan:
        peaks, s = plan.match(torch.from_numpy(buf).to(dev), torch.from_numpy(T).to(dev))
        torch.cuda.synchronize()
    ref, pk = oracle.ncc_match(img, T)
    assert np.max(np.abs(s[0].cpu().numpy() - ref)) <= TOL
    d = decode_peaks(peaks)
    assert (int(d["u"][0]), int(d["v"][0])) == (u0, v0)


def test_cfg2_split_k_bands_bitwise():
    """Split-K units + band shards: per-offset accumulation order is fixed per problem."""
    img, T, u0, v0 = synth.tm_inputs(2, k=2)
    full_peaks, full, info = run_match(img, T)
    assert "_s" in info["variant_name"]
    parts = []
    for r in range(2):
        pk, s, inf = run_match(img, T, shard=(r, 2))
        parts.append(s[0])
    np.testing.assert_array_equal(np.concatenate(parts, axis=0), full[0])


@pytest.mark.parametrize("cuda_cores", [True, False])
def test_concurrent_plans_on_two_streams(cuda_cores):
    """Two TM plans with different templates on two streams: the shared constant-bank
    template slot (CUDA-core path) is ordered by the library; tensor-core plans own their
    scratch; both results stay exact."""
    dev = torch.device("cuda", 0)
    imgs, Ts, refs = [], [], []
    for k in range(2):
        img, T, u0, v0 = synth.tm_inputs(2, k=10 + k)
        imgs.append(torch.from_numpy(img).to(dev))
        Ts.append(torch.from_numpy(T).to(dev))
        refs.append((u0, v0))
    streams = [torch.cuda.Stream(dev), torch.cuda.Stream(dev)]
    plans = [MatchPlan(1024, 1024, 128, 128, cuda_cores=cuda_cores) for _ in range(2)]
    try:
        outs = []
        for _ in range(3):
            for k in range(2):
                with torch.cuda.stream(streams[k]):
                    pk, _ = plans[k].match(imgs[k], Ts[k], stream=streams[k])
                    outs.append((k, pk))
        torch.cuda.synchronize()
        for k, pk in outs:
            d = decode_peaks(pk)
            assert (int(d["u"][0]), int(d["v"][0])) == refs[k]
            assert abs(float(d["score"][0]) - 1.0) <= TOL
    finally:
        for p in plans:
            p.close()


def test_c_example_runs_end_to_end(tmp_path):
    import os
    import subprocess
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    libdir = os.path.join(root, "paper_conf_ipps_moorelk13_b200")
    exe = tmp_path / "ncc_example"
    subprocess.check_call(["gcc", "-O2", "-I", os.path.join(root, "include"), os.path.join(root, "examples", "ncc_example.c"),
                           "-o", str(exe), "-L", libdir, "-lncc_b200", "-Wl,-rpath," + libdir])
    r = subprocess.run([str(exe)], capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stdout + r.stderr


@pytest.mark.parametrize("h,w", [(128, 128), (37, 300), (9, 5)])
def test_window_sum_forms_agree(h, w, monkeypatch):
    """Fused single-pass window sums vs the two-pass (row sums, column scan) form: bitwise equal
    scores on 2^-8-quantised inputs (every fp64 partial sum is exact there), and both within
    the oracle tolerance."""
    g = synth.rng(70 + h)
    img = synth.quantize(synth.uniform_image(300, 420, 71 + w))
    u, v = int(g.integers(0, 300 - h + 1)), int(g.integers(0, 420 - w + 1))
    T = np.ascontiguousarray(img[u:u + h, v:v + w])
    monkeypatch.setenv("NCC_BOX_FUSED", "1")  # windows >= 256 wide default to the two-pass form
    _, fused, info = run_match(img, T)
    monkeypatch.delenv("NCC_BOX_FUSED")
    monkeypatch.setenv("NCC_BOX_TWO_PASS", "1")
    _, two, info2 = run_match(img, T)
    assert info2["launches_per_call"] == info["launches_per_call"] + 1
    np.testing.assert_array_equal(fused, two)
    ref = oracle.ncc_surface(img, T)
    assert np.max(np.abs(fused[0] - ref)) <= TOL


@pytest.mark.parametrize("cuda_cores", [True, False])
def test_graph_replay_rotating_buffers(cuda_cores, tmp_path):
    """Execute calls replay captured CUDA graphs keyed by their pointer arguments (at most 4 per
    plan): rotating 6 buffer sets forces captures, replays and evictions; every call's peak is
    the planted one and the surfaces equal, bit for bit, a run launching kernel by kernel
    (NCC_NO_GRAPH=1 in a subprocess)."""
    import subprocess
    import sys
    import os
    dev = torch.device("cuda", 0)
    H, W, h, w = (256, 256, 32, 32)
    sets = []
    for k in range(6):
        img = synth.uniform_image(H, W, 9000 + k)
        T, u0, v0 = synth.planted_template(img, h, w, 9500 + k)
        sets.append((img, np.ascontiguousarray(T), u0, v0))
    np.save(tmp_path / "imgs.npy", np.stack([s[0] for s in sets]))
    np.save(tmp_path / "tmpls.npy", np.stack([s[1] for s in sets]))
    surfaces = {}
    with MatchPlan(H, W, h, w, write_surface=True, cuda_cores=cuda_cores) as plan:
        bufs = [(torch.from_numpy(s[0]).to(dev), torch.from_numpy(s[1]).to(dev)) for s in sets]
        for _ in range(3):
            for k, (di, dt) in enumerate(bufs):
                pk, sc = plan.match(di, dt)
                torch.cuda.synchronize()
                d = decode_peaks(pk)
                assert (int(d["u"][0]), int(d["v"][0])) == (sets[k][2], sets[k][3])
                surfaces[k] = sc[0].cpu().numpy()
    code = (
        "import sys, numpy as np, torch\n"
        f"sys.path.insert(0, {repr(os.getcwd())})\n"
        "from paper_conf_ipps_moorelk13_b200.api import MatchPlan\n"
        f"imgs = np.load({repr(str(tmp_path / 'imgs.npy'))}); ts = np.load({repr(str(tmp_path / 'tmpls.npy'))})\n"
        f"out = []\n"
        f"with MatchPlan({H}, {W}, {h}, {w}, write_surface=True, cuda_cores={cuda_cores}) as p:\n"
        "    for k in range(len(imgs)):\n"
        "        _, sc = p.match(torch.from_numpy(imgs[k]).cuda(), torch.from_numpy(ts[k]).cuda())\n"
        "        out.append(sc[0].cpu().numpy())\n"
        f"np.save({repr(str(tmp_path / 'direct.npy'))}, np.stack(out))\n")
    env = dict(os.environ, NCC_NO_GRAPH="1")
    subprocess.run([sys.executable, "-c", code], check=True, env=env, timeout=300)
    direct = np.load(tmp_path / "direct.npy")
    for k in range(6):
        np.testing.assert_array_equal(surfaces[k], direct[k])


@pytest.mark.parametrize("ssd", [False, True])
def test_tiny_one_launch_path(monkeypatch, ssd):
    """cfg1-sized problems run the whole path in one launch (tm_tiny_kernel): surfaces within
    the tolerance of the fp64 oracle (NCC; SSD relative to the energy scale), planted peaks
    exact, for a batch of frames, a band shard, and identical peaks with the general launch
    sequence (NCC_NO_TINY=1)."""
    dev = torch.device("cuda", 0)
    frames = [synth.tm_inputs(1, k=40 + k) for k in range(3)]
    T = frames[0][1]
    imgs = np.stack([frames[0][0]] + [f[0] for f in frames[1:]])
    score = 1 if ssd else 0
    d_img = torch.from_numpy(imgs).to(dev)
    d_t = torch.from_numpy(np.ascontiguousarray(T)).to(dev)
    outs = {}
    for tiny in (True, False):
        if not tiny:
            monkeypatch.setenv("NCC_NO_TINY", "1")
        with MatchPlan(64, 64, 16, 16, batch=3, write_surface=True, score=score) as plan:
            assert plan.info.variant_name.decode().startswith("tm_tiny") == tiny
            pk, sc = plan.match(d_img, d_t)
            pk, sc = plan.match(d_img, d_t)  # second call: keys / counters were reset by the first
            torch.cuda.synchronize()
            outs[tiny] = ({k: v.cpu().numpy() for k, v in decode_peaks(pk).items()}, sc.cpu().numpy())
    pk, sc = outs[True]
    for f in range(3):
        if ssd:
            ref, _ = oracle.ssd_match(imgs[f], T)
            scale = float((T.astype(np.float64) ** 2).sum() + (imgs[f].astype(np.float64) ** 2).sum() / 16)
            assert np.max(np.abs(sc[f] - ref)) <= 1e-5 * scale
        else:
            ref, _ = oracle.ncc_match(imgs[f], T)
            assert np.max(np.abs(sc[f] - ref)) <= TOL
    assert (int(pk["u"][0]), int(pk["v"][0])) == (frames[0][2], frames[0][3])
    for k in ("u", "v", "flags"):
        np.testing.assert_array_equal(pk[k], outs[False][0][k])
    # a band shard: global coordinates, rows of the band only
    monkeypatch.delenv("NCC_NO_TINY")
    with MatchPlan(64, 64, 16, 16, write_surface=True, shard_rank=1, shard_count=3) as plan:
        assert plan.info.variant_name.decode().startswith("tm_tiny")
        pk1, sc1 = plan.match(d_img[:1], d_t)
        torch.cuda.synchronize()
        u0, u1 = plan.info.u_begin, plan.info.u_end
        ref, _ = oracle.ncc_match(imgs[0], T)
        assert np.max(np.abs(sc1[0].cpu().numpy() - ref[u0:u1])) <= TOL


@pytest.mark.parametrize("shape,pinned", [((1024, 1024, 128, 128), True), ((1024, 1024, 128, 128), False),
                                          ((64, 64, 16, 16), True), ((200, 180, 24, 20), True)])
def test_host_path_alternating_buffers(shape, pinned):
    """Host entry point (the frames' and template's copies inside the captured launch sequence
    for pinned buffers, staged copies for pageable ones): alternating two input sets over
    several calls gives each set's planted peak (tensor-core, tiny and CUDA-core plans)."""
    H, W, h, w = shape
    sets = []
    for k in range(2):
        img = synth.uniform_image(H, W, 9100 + k)
        T, u0, v0 = synth.planted_template(img, h, w, 9200 + k)
        hi, ht = torch.from_numpy(img), torch.from_numpy(np.ascontiguousarray(T))
        if pinned:
            hi, ht = hi.pin_memory(), ht.pin_memory()
        sets.append((hi, ht, u0, v0))
    hp = torch.empty((1, 4), dtype=torch.int32).pin_memory()
    with MatchPlan(H, W, h, w) as plan:
        for _ in range(3):
            for hi, ht, u0, v0 in sets:
                plan.match_host(hi, ht, hp)
                torch.cuda.synchronize()
                d = decode_peaks(hp)
                assert (int(d["u"][0]), int(d["v"][0])) == (u0, v0)
                assert abs(float(d["score"][0]) - 1.0) <= TOL
