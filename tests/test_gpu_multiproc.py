"""Multi-process execution of the real sharded GPU path (north_star: offset bands
for one large match, frame pairs for PIV batches, only peaks / vectors gathered).

The round's hardware has one GPU, so two processes (a world_size-2 gloo group) share cuda:0:
each runs its shard through the CUDA library exactly as a torchrun rank would
(shard.sharded_match / shard.sharded_piv), then the 16-B peaks / 24-B vectors are gathered and
merged.  Checked: merged peaks and gathered vectors are bitwise equal to the one-process result,
band surfaces concatenate bitwise to the full surface, and both agree with the fp64 oracle
(planted peaks / shifts exact, sampled scores within 1e-4).
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.multiprocessing as mp

import oracle
import synth
from paper_conf_ipps_moorelk13_b200 import build as B

pytestmark = pytest.mark.gpu
TOL = 1e-4


@pytest.fixture(scope="module", autouse=True)
def _lib():
    B.build()


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _tm_worker(rank, world, port, out_dir):
    import torch.distributed as dist
    from paper_conf_ipps_moorelk13_b200 import shard
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        img, T, _, _ = synth.tm_inputs(5, k=21)
        dev = torch.device("cuda", 0)
        merged, band = shard.sharded_match(torch.from_numpy(img[None].copy()).to(dev), torch.from_numpy(T).to(dev),
                                           0, write_surface=True)
        torch.cuda.synchronize()
        np.save(os.path.join(out_dir, f"tm_peak{rank}.npy"), merged.cpu().numpy())
        np.save(os.path.join(out_dir, f"tm_band{rank}.npy"), band[0].cpu().numpy())
        # SSD bands merge with argmin
        merged_ssd, _ = shard.sharded_match(torch.from_numpy(img[None].copy()).to(dev), torch.from_numpy(T).to(dev),
                                            0, score=1)
        np.save(os.path.join(out_dir, f"tm_ssd{rank}.npy"), merged_ssd.cpu().numpy())
        dist.barrier()
    finally:
        dist.destroy_process_group()


def _piv_worker(rank, world, port, out_dir, total):
    import torch.distributed as dist
    from paper_conf_ipps_moorelk13_b200 import shard
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        a, b = shard.pair_range(total, rank, world)
        As, Bs = _piv_pairs(total)
        dev = torch.device("cuda", 0)
        allv = shard.sharded_piv(torch.from_numpy(As[a:b]).to(dev), torch.from_numpy(Bs[a:b]).to(dev), 64, 32, 32,
                                 total, 0)
        torch.cuda.synchronize()
        np.save(os.path.join(out_dir, f"piv{rank}.npy"), allv.cpu().numpy())
        dist.barrier()
    finally:
        dist.destroy_process_group()


def _piv_pairs(total):
    cv, specs = synth.piv_batch_from_canvases(4, total, canvases=2, k=5)
    As = np.stack([cv[ci][ay:ay + 2048, ax:ax + 2048] for (ci, ay, ax, by, bx, _) in specs])
    Bs = np.stack([cv[ci][by:by + 2048, bx:bx + 2048] for (ci, ay, ax, by, bx, _) in specs])
    return np.ascontiguousarray(As), np.ascontiguousarray(Bs)


def _spawn(target, args, world=2):
    ctx = mp.get_context("spawn")
    port = _free_port()
    procs = [ctx.Process(target=target, args=(r, world, port) + args) for r in range(world)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(timeout=600)
        assert p.exitcode == 0, p.exitcode


def test_two_process_band_sharded_cfg5_match(tmp_path):
    from paper_conf_ipps_moorelk13_b200.api import MatchPlan, decode_peaks
    _spawn(_tm_worker, (str(tmp_path),))
    img, T, u0, v0 = synth.tm_inputs(5, k=21)
    dev = torch.device("cuda", 0)
    with MatchPlan(4096, 4096, 512, 512, write_surface=True) as plan:
        pk, full = plan.match(torch.from_numpy(img).to(dev), torch.from_numpy(T).to(dev))
        torch.cuda.synchronize()
    one = pk.cpu().numpy()
    full = full[0].cpu().numpy()
    for r in range(2):
        np.testing.assert_array_equal(np.load(tmp_path / f"tm_peak{r}.npy"), one)  # bitwise, every rank
    bands = np.concatenate([np.load(tmp_path / f"tm_band{r}.npy") for r in range(2)], axis=0)
    np.testing.assert_array_equal(bands, full)
    d = decode_peaks(torch.from_numpy(one))
    assert (int(d["u"][0]), int(d["v"][0])) == (u0, v0)
    # band boundary rows and a few samples against the fp64 oracle
    g = synth.rng(2100)
    us = np.concatenate([[1792, 1791, u0, 0, 3584], g.integers(0, 3585, 11)])
    vs = np.concatenate([[0, 3584, v0, 17, 3584], g.integers(0, 3585, 11)])
    assert np.max(np.abs(full[us, vs] - oracle.ncc_at(img, T, us, vs))) <= TOL
    ssd = decode_peaks(torch.from_numpy(np.load(tmp_path / "tm_ssd0.npy")))
    assert (int(ssd["u"][0]), int(ssd["v"][0])) == (u0, v0)


def test_two_process_pair_sharded_piv(tmp_path):
    from paper_conf_ipps_moorelk13_b200.api import PivPlan, decode_vectors
    total = 5  # unequal shards (3 + 2 pairs)
    _spawn(_piv_worker, (str(tmp_path), total))
    As, Bs = _piv_pairs(total)
    dev = torch.device("cuda", 0)
    with PivPlan(2048, 2048, 64, 32, 32, pairs=total) as plan:
        vec, _ = plan.correlate(torch.from_numpy(As).to(dev), torch.from_numpy(Bs).to(dev))
        torch.cuda.synchronize()
    one = vec.cpu().numpy()
    for r in range(2):
        np.testing.assert_array_equal(np.load(tmp_path / f"piv{r}.npy"), one)
    d = {k: v.numpy() for k, v in decode_vectors(torch.from_numpy(one)).items()}
    _, specs = synth.piv_batch_from_canvases(4, total, canvases=2, k=5)
    for p, s in enumerate(specs):
        dy, dx = s[5]
        assert np.all(d["iy"][p] == dy) and np.all(d["ix"][p] == dx)
    kys, kxs = [0, 30, 60], [60, 7, 0]
    ref = oracle.piv_windows(As[4], Bs[4], 64, 64, 32, 32, 32, 32, kys, kxs)
    for i, (ky, kx) in enumerate(zip(kys, kxs)):
        assert abs(d["score"][4, ky, kx] - ref["score"][i]) <= TOL
        assert d["flags"][4, ky, kx] == ref["flags"][i]
