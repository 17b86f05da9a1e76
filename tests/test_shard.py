"""Host-side sharding logic (no GPU): band/pair partitions, the peak merge with the
single-GPU tie rule, and the gather path over a real world_size-2 gloo process group."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_ipps_moorelk13_b200 import shard


@pytest.mark.parametrize("U,n", [(3585, 8), (897, 8), (49, 3), (10, 10), (7, 3), (1000, 7)])
def test_band_ranges_partition(U, n):
    rows = []
    for r in range(n):
        a, b = shard.band_range(U, r, n)
        assert b > a
        rows.extend(range(a, b))
    assert rows == list(range(U))


def test_pair_ranges_partition():
    got = [shard.pair_range(256, r, 8) for r in range(8)]
    assert got == [(32 * r, 32 * r + 32) for r in range(8)]
    got = [shard.pair_range(10, r, 4) for r in range(4)]
    assert sum(b - a for a, b in got) == 10 and got[0][0] == 0 and got[-1][1] == 10


def _records_from_surface(S, bands):
    """Per-band argmax records the way a GPU band would report them (same tie rule)."""
    V = S.shape[1]
    recs = []
    for (a, b) in bands:
        sub = S[a:b]
        k = int(np.argmax(sub))  # numpy: first maximum = smallest linear index
        u, v = a + k // V, k % V
        recs.append([np.float32(sub.ravel()[k]).view(np.int32), u, v, 0])
    return torch.tensor(np.array(recs, dtype=np.int32))


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_merge_equals_global_argmax_with_ties(seed):
    g = np.random.default_rng(seed)
    S = np.round(0.9 * g.random((37, 23)), 2).astype(np.float32)  # coarse values -> many exact ties
    S[5, 7] = S[30, 1] = S[20, 22] = 1.0
    for n in (1, 2, 3, 5):
        bands = [shard.band_range(37, r, n) for r in range(n)]
        merged = shard.merge_peaks(_records_from_surface(S, bands)[:, None, :], 23)
        k = int(np.argmax(S))
        assert (int(merged[0, 1]), int(merged[0, 2])) == (k // 23, k % 23) == (5, 7)


def test_merge_ssd_takes_minimum_and_ties_smallest_index():
    """SSD peaks (argmin): the band merge must keep the smallest SSD, ties -> smallest u*V+v."""
    V = 10
    recs = torch.tensor(np.array([[np.float32(3.5).view(np.int32), 0, 4, 0],
                                  [np.float32(0.25).view(np.int32), 7, 1, 0],
                                  [np.float32(0.25).view(np.int32), 5, 9, 0],
                                  [np.float32(9.0).view(np.int32), 9, 0, 0]], dtype=np.int32))
    m = shard.merge_peaks(recs[:, None, :], V, ssd=True)
    assert (int(m[0, 1]), int(m[0, 2])) == (5, 9)
    m = shard.merge_peaks(recs[:, None, :], V, ssd=False)
    assert (int(m[0, 1]), int(m[0, 2])) == (9, 0)


def test_peak_keys_order_matches_score_then_index():
    """Packed keys sort like (score desc, index asc) over negative, zero and positive scores."""
    g = np.random.default_rng(3)
    sc = np.concatenate([g.standard_normal(200).astype(np.float32), [0.0, 0.0, 1.0, 1.0, -1.0]]).astype(np.float32)
    us = g.integers(0, 50, sc.size)
    vs = g.integers(0, 30, sc.size)
    recs = torch.tensor(np.stack([sc.view(np.int32), us, vs, np.zeros_like(us)], 1).astype(np.int32))
    k = shard.peak_keys(recs, 30).numpy()
    order = np.argsort(-k, kind="stable")
    ref = sorted(range(sc.size), key=lambda i: (-float(sc[i]), us[i] * 30 + vs[i]))
    # equal (score, index) pairs are interchangeable; compare the sorted tuples
    assert [(float(sc[i]), us[i] * 30 + vs[i]) for i in order] == [(float(sc[i]), us[i] * 30 + vs[i]) for i in ref]


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, S, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        U, V = S.shape
        a, b = shard.band_range(U, rank, world)
        rec = _records_from_surface(S, [(a, b)])  # (1, 4): one frame
        allp = shard.gather_results(rec)          # (world, 1, 4)
        merged = shard.merge_peaks(allp, V)
        # PIV: unequal pair counts gathered in pair order
        P = 5
        pa, pb = shard.pair_range(P, rank, world)
        vec = torch.arange(pa, pb, dtype=torch.int32).reshape(-1, 1, 1, 1).expand(-1, 2, 3, 6).contiguous()
        counts = [shard.pair_range(P, r, world)[1] - shard.pair_range(P, r, world)[0] for r in range(world)]
        allv = shard.gather_vectors(vec, counts)
        q.put((rank, merged.numpy().tolist(), allv[:, 0, 0, 0].numpy().tolist()))
    finally:
        dist.destroy_process_group()


def test_gloo_world2_gather_and_merge():
    g = np.random.default_rng(7)
    S = np.round(0.9 * g.random((41, 19)), 2).astype(np.float32)
    S[33, 4] = S[35, 2] = 1.0  # global peak lives in rank 1's band; a tie after it
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, S, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in range(2)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    k = int(np.argmax(S))
    for rank, merged, order in res:
        assert (merged[0][1], merged[0][2]) == (k // 19, k % 19) == (33, 4)
        assert order == [0, 1, 2, 3, 4]
