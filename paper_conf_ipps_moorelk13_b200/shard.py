"""Multi-GPU sharding of the NCC hot path (BASELINE north_star: "offset
bands for a single large match ... frame pairs for PIV batches, with an NCCL gather over
NVLink only for peak and vector results").

One process per GPU (torchrun).  Data-path work never crosses GPUs: each rank computes its
band of offset rows (TM) or its contiguous range of frame pairs (PIV) with the C ABI, then
only the results move -- 16-B ncc_peak records or 24-B piv_vector records -- through
torch.distributed (NCCL over NVLink on the B200 box; gloo in the CPU tests).

The merge uses the same tie rule as inside one GPU: max score, ties -> smallest global
linear offset index u*V + v (SURVEY 8(c) reading 5), so an n-GPU peak equals the 1-GPU peak;
per-offset accumulation order does not depend on the band, so scores are bitwise equal.
"""
from __future__ import annotations

import torch
import torch.distributed as dist


def band_range(U: int, rank: int, world: int) -> tuple[int, int]:
    """Offset rows of rank's band -- the same rule as ncc_plan_create (balanced, contiguous)."""
    return (rank * U) // world, ((rank + 1) * U) // world


def pair_range(P: int, rank: int, world: int) -> tuple[int, int]:
    """Frame pairs of rank's PIV shard (balanced, contiguous)."""
    return (rank * P) // world, ((rank + 1) * P) // world


def peak_keys(peaks: torch.Tensor, V: int, ssd: bool = False) -> torch.Tensor:
    """int32 (..., 4) ncc_peak records -> int64 keys ordered like the kernels' packed 64-bit key
    (csrc make_key): high 32 bits = order-preserving image of the fp32 score (of -score for SSD,
    whose peak is the minimum), low 32 bits = 0xFFFFFFFF - (u*V + v), so the largest key is the
    best score with ties going to the smallest global linear offset index.  Shifted by -2^63
    so the unsigned key order is the signed int64 order."""
    p = peaks.reshape(-1, 4) if peaks.dim() == 1 else peaks
    score = p[..., 0].view(torch.float32)
    if ssd:
        score = -score
    b = score.view(torch.int32).to(torch.int64) & 0xFFFFFFFF
    o = torch.where(b >= 0x80000000, (~b) & 0xFFFFFFFF, b | 0x80000000)
    lin = p[..., 1].to(torch.int64) * V + p[..., 2].to(torch.int64)
    return (o - 0x80000000) * (1 << 32) + (0xFFFFFFFF - lin)


def merge_peaks(peaks: torch.Tensor, V: int, ssd: bool = False) -> torch.Tensor:
    """peaks: int32 (world, batch, 4) ncc_peak records -> (batch, 4) merged records.

    One max over the packed keys per frame (the kernels' own tie rule: best score -- max for
    NCC, min for SSD -- then the smallest u*V+v).  Records are selected, never recomputed; no
    host synchronisation (works on the device for NCCL-gathered records).
    """
    p = peaks.reshape(peaks.shape[0], -1, 4)
    best = torch.argmax(peak_keys(p, V, ssd), dim=0)  # (batch,) rank holding each frame's peak
    return p[best, torch.arange(p.shape[1], device=p.device)]


def gather_results(local: torch.Tensor, group=None) -> torch.Tensor:
    """All-gather equally shaped per-rank result records -> (world, *local.shape)."""
    world = dist.get_world_size(group)
    if dist.get_backend(group) == "nccl":
        out = torch.empty((world,) + tuple(local.shape), dtype=local.dtype, device=local.device)
        dist.all_gather_into_tensor(out, local.contiguous(), group=group)
        return out
    # gloo (CPU tests, or several ranks sharing one GPU): host tensors
    src = local.detach().cpu().contiguous()
    parts = [torch.empty_like(src) for _ in range(world)]
    dist.all_gather(parts, src, group=group)
    return torch.stack(parts).to(local.device)


def gather_vectors(local: torch.Tensor, counts: list[int], group=None) -> torch.Tensor:
    """PIV: gather (pairs_r, Ky, Kx, 6) records of unequal pair counts -> concatenated in pair order."""
    world = dist.get_world_size(group)
    mx = max(counts)
    pad = torch.zeros((mx,) + tuple(local.shape[1:]), dtype=local.dtype, device=local.device)
    pad[: local.shape[0]] = local
    allv = gather_results(pad, group)
    return torch.cat([allv[r, : counts[r]] for r in range(world)], dim=0)


def sharded_match(images: torch.Tensor, tmpl: torch.Tensor, device: int, group=None, write_surface=False,
                  score: int = 0):
    """Single large match split by offset-row bands over the process group.

    Every rank holds the full frame(s) (it reads only rows [u0, u1+h-1)); returns the merged
    (batch, 4) peak records on every rank, plus this rank's surface band if requested.
    """
    from .api import MatchPlan
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    B, H, W = images.shape
    h, w = tmpl.shape
    with MatchPlan(H, W, h, w, batch=B, device=device, shard_rank=rank, shard_count=world,
                   write_surface=write_surface, score=score) as plan:
        peaks, scores = plan.match(images, tmpl)
        V = plan.info.V
    allp = gather_results(peaks, group)
    return merge_peaks(allp, V, ssd=score == 1), scores


def sharded_piv(frames_a: torch.Tensor, frames_b: torch.Tensor, win, search, step, total_pairs: int, device: int,
                group=None):
    """PIV batch split by frame pairs: frames_* hold only this rank's pairs (pair_range)."""
    from .api import PivPlan
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    counts = [pair_range(total_pairs, r, world)[1] - pair_range(total_pairs, r, world)[0] for r in range(world)]
    P, H, W = frames_a.shape
    assert P == counts[rank]
    with PivPlan(H, W, win, search, step, pairs=P, device=device) as plan:
        vec, _ = plan.correlate(frames_a, frames_b)
    return gather_vectors(vec, counts, group)
