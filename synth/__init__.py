"""Seeded synthetic inputs shared by the oracle tests, the GPU parity tests and bench.py.

This module holds NO arithmetic of the method (no correlation, no sums over windows,
no peak search): it only draws images, templates and particle-image pairs with the
shapes and statistics of the paper's workloads (recipe restated
in DESIGN.md "Input recipe").  Both sides (oracle, CUDA path) receive the same arrays.

Generators use numpy PCG64 with explicit seeds (seed = cfg_index*1000 + k).
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np

# The five BASELINE.json configurations.
CONFIGS = {
    1: dict(kind="tm", H=64, W=64, h=16, w=16),
    2: dict(kind="tm", H=1024, W=1024, h=128, w=128),
    3: dict(kind="piv", H=1024, W=1024, h=32, w=32, m=16, step=16, pairs=1, max_shift=14),
    4: dict(kind="piv", H=2048, W=2048, h=64, w=64, m=32, step=32, pairs=256, max_shift=30),
    5: dict(kind="tm", H=4096, W=4096, h=512, w=512),
}


def rng(seed: int) -> np.random.Generator:
    return np.random.Generator(np.random.PCG64(seed))


def uniform_image(H: int, W: int, seed: int) -> np.ndarray:
    """I ~ U[0,1) fp32."""
    return rng(seed).random((H, W), dtype=np.float32)


def quantize(a: np.ndarray, bits: int = 8) -> np.ndarray:
    """Round to multiples of 2^-bits (inputs whose fp64 window sums are exact)."""
    q = float(1 << bits)
    return (np.floor(np.asarray(a, dtype=np.float64) * q) / q).astype(np.float32)


def _gauss_kernel(sigma: float) -> np.ndarray:
    r = int(np.ceil(4 * sigma))
    x = np.arange(-r, r + 1, dtype=np.float64)
    k = np.exp(-0.5 * (x / sigma) ** 2)
    return k / k.sum()


def smooth_image(H: int, W: int, seed: int, sigma: float = 4.0, mean: float = 0.5, sd: float = 0.1) -> np.ndarray:
    """Gaussian-filtered N(0,1) noise rescaled to (mean, sd): the cancellation-stress
    input of SURVEY.md 8(d) (large mean, small variance)."""
    g = rng(seed).standard_normal((H, W))
    k = _gauss_kernel(sigma)
    r = len(k) // 2
    gp = np.pad(g, r, mode="wrap")
    # separable filtering (input generation only)
    t = np.zeros((H + 2 * r, W))
    for i, kv in enumerate(k):
        t += kv * gp[:, i:i + W]
    s = np.zeros((H, W))
    for i, kv in enumerate(k):
        s += kv * t[i:i + H, :]
    s = (s - s.mean()) / s.std()
    return (mean + sd * s).astype(np.float32)


def planted_template(img: np.ndarray, h: int, w: int, seed: int) -> tuple[np.ndarray, int, int]:
    """Cut an h x w template out of img at a seeded origin (u0, v0): it scores 1 there."""
    H, W = img.shape
    g = rng(seed)
    u0 = int(g.integers(0, H - h + 1))
    v0 = int(g.integers(0, W - w + 1))
    return np.ascontiguousarray(img[u0:u0 + h, v0:v0 + w]), u0, v0


def tm_inputs(cfg: int, k: int = 0, smooth: bool = False) -> tuple[np.ndarray, np.ndarray, int, int]:
    c = CONFIGS[cfg]
    seed = cfg * 1000 + k
    img = smooth_image(c["H"], c["W"], seed) if smooth else uniform_image(c["H"], c["W"], seed)
    T, u0, v0 = planted_template(img, c["h"], c["w"], seed + 500)
    return img, T, u0, v0


# ----------------------------------------------------------------------------------
# Particle images (PIV): Gaussian particles, d_p = 2.6 px (e^-2 diameter, sigma = d_p/4),
# 0.05 particles per pixel, intensity U[0.5, 1], background 0.
# ----------------------------------------------------------------------------------

def render_particles(H: int, W: int, py: np.ndarray, px: np.ndarray, amp: np.ndarray,
                     d_p: float = 2.6) -> np.ndarray:
    sigma = d_p / 4.0
    img = np.zeros((H, W), dtype=np.float64)
    r = int(np.ceil(3 * sigma))
    cy = np.floor(py).astype(np.int64)
    cx = np.floor(px).astype(np.int64)
    for oy in range(-r, r + 2):
        for ox in range(-r, r + 2):
            yy = cy + oy
            xx = cx + ox
            ok = (yy >= 0) & (yy < H) & (xx >= 0) & (xx < W)
            val = amp * np.exp(-((yy - py) ** 2 + (xx - px) ** 2) / (2 * sigma * sigma))
            np.add.at(img, (yy[ok], xx[ok]), val[ok])
    return img


def particle_canvas(H: int, W: int, seed: int, density: float = 0.05, d_p: float = 2.6) -> np.ndarray:
    g = rng(seed)
    n = int(round(density * H * W))
    py = g.random(n) * H
    px = g.random(n) * W
    amp = 0.5 + 0.5 * g.random(n)
    return render_particles(H, W, py, px, amp, d_p)


@dataclass
class PivPair:
    A: np.ndarray
    B: np.ndarray
    shift: tuple  # (dy, dx): B(y+dy, x+dx) ~= A(y, x)


def particle_pair_integer(H: int, W: int, dy: int, dx: int, seed: int, noise: float = 0.0,
                          density: float = 0.05) -> PivPair:
    """Exact integer translate: A and B are crops of one padded canvas so that
    B[y+dy, x+dx] == A[y, x] wherever both are defined."""
    M = max(abs(dy), abs(dx)) + 8
    C = particle_canvas(H + 2 * M, W + 2 * M, seed, density)
    A = C[M:M + H, M:M + W]
    B = C[M - dy:M - dy + H, M - dx:M - dx + W]
    if noise > 0:
        g = rng(seed + 77)
        A = A + noise * g.standard_normal(A.shape)
        B = B + noise * g.standard_normal(B.shape)
    return PivPair(np.ascontiguousarray(A, dtype=np.float32), np.ascontiguousarray(B, dtype=np.float32), (dy, dx))


def particle_pair_subpixel(H: int, W: int, dy: float, dx: float, seed: int, density: float = 0.05) -> PivPair:
    """Continuous shift: particles re-rendered at p + (dy, dx) in B."""
    g = rng(seed)
    M = int(np.ceil(max(abs(dy), abs(dx)))) + 8
    n = int(round(density * (H + 2 * M) * (W + 2 * M)))
    py = g.random(n) * (H + 2 * M) - M
    px = g.random(n) * (W + 2 * M) - M
    amp = 0.5 + 0.5 * g.random(n)
    A = render_particles(H, W, py, px, amp)
    B = render_particles(H, W, py + dy, px + dx, amp)
    return PivPair(A.astype(np.float32), B.astype(np.float32), (dy, dx))


def piv_shift_for_pair(cfg: int, p: int) -> tuple[int, int]:
    """Planted integer shift of pair p of config cfg, |d| <= max_shift."""
    c = CONFIGS[cfg]
    g = rng(cfg * 1000 + 900 + p)
    s = c["max_shift"]
    return int(g.integers(-s, s + 1)), int(g.integers(-s, s + 1))


def piv_batch_from_canvases(cfg: int, pairs: int, canvases: int = 4, k: int = 0):
    """Pairs cropped from a few large rendered canvases (SURVEY 8(d) cfg 4 recipe).

    Returns (canvas_list, specs) where specs[p] = (canvas index, ay, ax, by, bx, (dy, dx)):
    A = canvas[ay:ay+H, ax:ax+W], B = canvas[by:by+H, bx:bx+W], with
    B[y+dy, x+dx] == A[y, x].  Crops are materialised by the caller (on the device for
    the big batch) so the host never holds all pairs.
    """
    c = CONFIGS[cfg]
    H, W, s = c["H"], c["W"], c["max_shift"]
    M = s + 8
    CH, CW = H + 2 * M + 64, W + 2 * M + 64
    cv = [particle_canvas(CH, CW, cfg * 1000 + 700 + k * 16 + i).astype(np.float32) for i in range(canvases)]
    specs = []
    for p in range(pairs):
        g = rng(cfg * 1000 + 800 + p)
        dy, dx = piv_shift_for_pair(cfg, p)
        ay = M + int(g.integers(0, 65))
        ax = M + int(g.integers(0, 65))
        specs.append((p % canvases, ay, ax, ay - dy, ax - dx, (dy, dx)))
    return cv, specs
