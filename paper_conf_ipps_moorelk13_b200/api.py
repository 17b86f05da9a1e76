"""User-facing wrappers over the C ABI: plans as context managers, torch tensors in and out.

Marshalling only -- allocation of output tensors and pointer/stream passing.  Results are
raw ncc_peak / piv_vector records held in torch int32 tensors; decode_* turn them into
named fields (views, no arithmetic of the method).
"""
from __future__ import annotations

from dataclasses import dataclass

import torch

from . import _native as N


def decode_peaks(raw: torch.Tensor) -> dict:
    """raw: int32 (batch, 4) ncc_peak records -> dict of tensors."""
    r = raw.reshape(-1, 4)
    return {"score": r[:, 0].view(torch.float32), "u": r[:, 1], "v": r[:, 2], "flags": r[:, 3]}


def decode_vectors(raw: torch.Tensor) -> dict:
    """raw: int32 (..., 6) piv_vector records -> dict of tensors (same leading shape)."""
    return {"iy": raw[..., 0], "ix": raw[..., 1], "dy": raw[..., 2].view(torch.float32),
            "dx": raw[..., 3].view(torch.float32), "score": raw[..., 4].view(torch.float32), "flags": raw[..., 5]}


class _Plan:
    def __init__(self, problem: N.NccProblem, device: int):
        self.problem = problem
        self.device = int(device)
        self.handle = N.ncc_plan_create(problem, self.device)
        self.info = N.ncc_plan_query(self.handle)

    def close(self):
        if self.handle:
            N.ncc_plan_destroy(self.handle)
            self.handle = None

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def timing(self) -> N.NccTiming:
        return N.ncc_plan_timing(self.handle)

    def _stream(self, stream):
        return N._stream(stream, torch.device("cuda", self.device))


class MatchPlan(_Plan):
    """Template matching: corr2 at every valid offset of each frame (Listing 5.1)."""

    def __init__(self, H, W, h, w, batch=1, device=0, shard_rank=0, shard_count=1, write_surface=False,
                 generic=False, timing=False, image_pitch=None, score=N.NCC_SCORE_NCC, n_templates=0, roi=None,
                 cuda_cores=False):
        """roi=(roi_h, roi_w) with n_templates >= 1 selects ROI mode (match_rois); cuda_cores=True never
        uses the tensor-core numerator (the library picks it by a cost model otherwise)."""
        flags = (N.NCC_F_WRITE_SURFACE if write_surface else 0) | (N.NCC_F_GENERIC_KERNEL if generic else 0) | \
                (N.NCC_F_TIMING if timing else 0) | (N.NCC_F_CUDA_CORES if cuda_cores else 0)
        rh, rw = roi if roi is not None else (0, 0)
        super().__init__(N.make_problem(N.NCC_MODE_MATCH, H, W, image_pitch, h, w, batch=batch,
                                        shard_rank=shard_rank, shard_count=shard_count, flags=flags,
                                        score=score, n_templates=n_templates, roi_h=rh, roi_w=rw), device)
        self.write_surface = write_surface

    @property
    def band_rows(self):
        return self.info.u_end - self.info.u_begin

    def match(self, images: torch.Tensor, tmpl: torch.Tensor, stream=None, peaks=None, scores=None):
        p = self.problem
        dev = torch.device("cuda", self.device)
        assert images.is_cuda and images.dtype == torch.float32 and tmpl.dtype == torch.float32
        if peaks is None:
            peaks = torch.empty((p.batch, 4), dtype=torch.int32, device=dev)
        if self.write_surface and scores is None:
            scores = torch.empty((p.batch, self.band_rows, self.info.V), dtype=torch.float32, device=dev)
        N.ncc_match(self.handle, images, tmpl, tmpl.stride(0), scores, peaks, self._stream(stream))
        return peaks, scores

    def match_rois(self, images: torch.Tensor, tmpls: torch.Tensor, rois: torch.Tensor, stream=None, peaks=None,
                   scores=None):
        """images (batch, H, pitch); tmpls (T, h, w); rois int32 (batch, T, 2) origins (u0, v0)."""
        p = self.problem
        dev = torch.device("cuda", self.device)
        T = max(1, p.n_templates)
        if peaks is None:
            peaks = torch.empty((p.batch, T, 4), dtype=torch.int32, device=dev)
        if self.write_surface and scores is None:
            scores = torch.empty((p.batch, T, p.roi_h, p.roi_w), dtype=torch.float32, device=dev)
        N.ncc_match_rois(self.handle, images, tmpls, tmpls.stride(1), rois, scores, peaks, self._stream(stream))
        return peaks, scores

    def match_host(self, h_images: torch.Tensor, h_tmpl: torch.Tensor, h_peaks: torch.Tensor, h_scores=None,
                   stream=None):
        N.ncc_match_host(self.handle, h_images, h_tmpl, h_tmpl.stride(0), h_scores, h_peaks, self._stream(stream))
        return h_peaks


class PivPlan(_Plan):
    """PIV: per-window NCC over a search range, peak + 3-point sub-pixel fit (Figs 5.8-5.12)."""

    def __init__(self, H, W, win, search, step, pairs=1, device=0, subpix=N.NCC_SUBPIX_GAUSS3, generic=False,
                 timing=False, image_pitch=None, score=N.NCC_SCORE_NCC):
        wh, ww = (win, win) if isinstance(win, int) else win
        my, mx = (search, search) if isinstance(search, int) else search
        sy, sx = (step, step) if isinstance(step, int) else step
        flags = (N.NCC_F_GENERIC_KERNEL if generic else 0) | (N.NCC_F_TIMING if timing else 0)
        super().__init__(N.make_problem(N.NCC_MODE_PIV, H, W, image_pitch, wh, ww, my, mx, sy, sx, batch=pairs,
                                        flags=flags, subpix=subpix, score=score), device)

    @property
    def grid(self):
        return self.info.Ky, self.info.Kx

    def correlate(self, A: torch.Tensor, B: torch.Tensor, stream=None, vectors=None, scores=False):
        p = self.problem
        dev = torch.device("cuda", self.device)
        Ky, Kx = self.grid
        if vectors is None:
            vectors = torch.empty((p.batch, Ky, Kx, 6), dtype=torch.int32, device=dev)
        sc = None
        if scores:
            sc = torch.empty((p.batch, Ky, Kx, 2 * p.search_y + 1, 2 * p.search_x + 1), dtype=torch.float32,
                             device=dev)
        N.piv_correlate_ex(self.handle, A, B, sc, vectors, self._stream(stream))
        return vectors, sc

    def correlate_host(self, h_A, h_B, h_vectors, stream=None):
        N.piv_correlate_host(self.handle, h_A, h_B, h_vectors, self._stream(stream))
        return h_vectors
