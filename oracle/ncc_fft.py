"""Independent fp64 FFT route to the full NCC surface.

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).  This is a second, independent
oracle route used to (a) cross-check the brute-force C oracle and (b) give full-size
(cfg 2 / cfg 5) reference surfaces that the brute-force oracle would take hours for.
It follows the same definition -- corr2 / Pearson per valid offset (Fig 5.1 caption
P:132-137, Listing 5.1 caption P:250-251) -- through a different algebra:

    num(u,v) = sum_ij (T - Tbar)[i,j] * I[u+i, v+j]          (FFT cross-correlation)
    S1, S2   = window sums of I and I^2                         (fp64 summed-area table)
    sw       = S2 - S1^2 / n ,  st = sum (T - Tbar)^2
    score    = num / sqrt(st * sw), 0 if st <= 1e-10 sum T^2 or sw <= 1e-10 S2

The identity sum (T-Tbar)(W-Wbar) = sum (T-Tbar) W holds because sum (T-Tbar) = 0
(Fig 5.2/5.3 captions P:138-153: A_C = template minus its average).  A library FFT
is a step here, as the oracle rules allow; nothing is shared with the CUDA path.
"""
from __future__ import annotations

import numpy as np


def window_sums(img: np.ndarray, h: int, w: int) -> tuple[np.ndarray, np.ndarray]:
    """S1, S2 over every valid h x w window via fp64 summed-area tables."""
    I = np.asarray(img, dtype=np.float64)
    H, W = I.shape
    sat1 = np.zeros((H + 1, W + 1))
    sat2 = np.zeros((H + 1, W + 1))
    sat1[1:, 1:] = I.cumsum(0).cumsum(1)
    sat2[1:, 1:] = (I * I).cumsum(0).cumsum(1)

    def box(s):
        return s[h:, w:] - s[:-h, w:] - s[h:, :-w] + s[:-h, :-w]

    return box(sat1), box(sat2)


def ncc_surface_fft(img: np.ndarray, tmpl: np.ndarray) -> np.ndarray:
    I = np.asarray(img, dtype=np.float64)
    T = np.asarray(tmpl, dtype=np.float64)
    H, W = I.shape
    h, w = T.shape
    U, V = H - h + 1, W - w + 1
    n = h * w
    Tc = T - T.sum() / n
    st = float((Tc * Tc).sum())
    sumT2 = float((T * T).sum())
    FI = np.fft.rfft2(I)
    FT = np.fft.rfft2(Tc, s=(H, W))
    num = np.fft.irfft2(FI * np.conj(FT), s=(H, W))[:U, :V]
    S1, S2 = window_sums(I, h, w)
    sw = S2 - S1 * S1 / n
    out = np.zeros((U, V))
    if st <= 1e-10 * sumT2:
        return out
    ok = sw > 1e-10 * S2
    out[ok] = num[ok] / np.sqrt(st * sw[ok])
    return out
