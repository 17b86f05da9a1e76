#!/usr/bin/env python
"""Benchmark of the B200 NCC hot path (BASELINE.json metric: NCC offsets/s & PIV vectors/s,
% of the FP32 roofline).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--workload cfg2|cfg1|cfg3|cfg4|cfg5]
                    [--impl ours|reference] [--no-secondary]

A step is one pass of the whole hot path over one batch of synthetic input: for TM
(cfg1/2/5) template prep -> fp64 window sums -> numerator + fused normalise/argmax ->
peak finalise; for PIV (cfg3/4) window sums -> batched
correlation + peak + sub-pixel (a2, a6, a7).  Default workload = configs[1] (cfg2:
128x128 template in a 1024x1024 image, 804,609 offsets).  N > 1 (torchrun): every rank
runs its own frame(s) (weak scaling, no data-path collective); the per-rank results
(16-B peaks / 24-B vectors) are gathered to rank 0 with NCCL over NVLink.

--impl reference times the fp64 CPU oracle (oracle/, the only reference that exists for
this paper) on a bounded sample of the same workload, on rank 0 only.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import synth  # noqa: E402

L2_FLUSH_BYTES = 512 << 20  # > 126 MB L2


# ----------------------------------------------------------------------------- helpers
def dist_env():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


def physical_gpu_index(local):
    vis = os.environ.get("CUDA_VISIBLE_DEVICES")
    if vis:
        ids = [x.strip() for x in vis.split(",") if x.strip()]
        if local < len(ids):
            return ids[local]
    return str(local)


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled DURING the timed region."""
    FIELDS = ["clocks.sm", "clocks.max.sm", "power.draw", "clocks_event_reasons.hw_slowdown",
              "clocks_event_reasons.hw_thermal_slowdown", "clocks_event_reasons.sw_thermal_slowdown",
              "clocks_event_reasons.sw_power_cap"]

    def __init__(self, gpu):
        self.gpu = gpu
        self.rows = []
        self.proc = None

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.gpu), "--query-gpu=" + ",".join(self.FIELDS),
                 "--format=csv,noheader,nounits", "-lms", "100"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.th = threading.Thread(target=self._read, daemon=True)
            self.th.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            parts = [p.strip() for p in line.split(",")]
            if len(parts) == len(self.FIELDS):
                self.rows.append(parts)

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"]}
        time.sleep(0.25)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        self.th.join(timeout=2)
        sm = [float(r[0]) for r in self.rows if r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()]
        loaded = [s for s in sm if s > 600] or sm
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in self.rows for i in range(4) if r[3 + i].lower() == "active"})
        return {"sm_mhz": statistics.median(loaded) if loaded else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.rows)}


def cpu_cores():
    try:
        return len(os.sched_getaffinity(0))
    except Exception:
        return os.cpu_count() or 1


# ----------------------------------------------------------------------------- workloads
def tm_workload(cfg, rank):
    c = synth.CONFIGS[cfg]
    img, T, u0, v0 = synth.tm_inputs(cfg, k=rank)
    return dict(kind="tm", cfg=cfg, img=img, T=T, planted=(u0, v0), H=c["H"], W=c["W"], h=c["h"], w=c["w"])


def piv_workload(cfg, rank, world):
    c = synth.CONFIGS[cfg]
    pairs = c["pairs"]
    per = max(1, pairs // world) if cfg == 4 else pairs
    return dict(kind="piv", cfg=cfg, H=c["H"], W=c["W"], h=c["h"], w=c["w"], m=c["m"], step=c["step"], pairs=per,
                rank=rank)


def piv_frames_device(wl, dev, torch):
    """Materialise the rank's frame pairs on the device (crops of a few rendered canvases)."""
    cfg, H, W, P = wl["cfg"], wl["H"], wl["W"], wl["pairs"]
    if cfg == 3:
        dy, dx = synth.piv_shift_for_pair(3, wl["rank"])
        p = synth.particle_pair_integer(H, W, dy, dx, seed=3000 + wl["rank"])
        A = torch.from_numpy(p.A[None].copy()).to(dev)
        B = torch.from_numpy(p.B[None].copy()).to(dev)
        return A, B, [(dy, dx)]
    cv, specs = synth.piv_batch_from_canvases(cfg, P, canvases=4, k=wl["rank"])
    cvd = [torch.from_numpy(c).to(dev) for c in cv]
    A = torch.empty((P, H, W), dtype=torch.float32, device=dev)
    B = torch.empty((P, H, W), dtype=torch.float32, device=dev)
    for i, (ci, ay, ax, by, bx, _) in enumerate(specs):
        A[i].copy_(cvd[ci][ay:ay + H, ax:ax + W])
        B[i].copy_(cvd[ci][by:by + H, bx:bx + W])
    del cvd
    return A, B, [s[5] for s in specs]


# ----------------------------------------------------------------------------- reference arm
def run_reference(args, wl_cfg):
    """fp64 CPU oracle timed on this host (rank 0 only), bounded sample per step."""
    import oracle
    cores = cpu_cores()
    os.environ.setdefault("OMP_NUM_THREADS", str(cores))
    c = synth.CONFIGS[wl_cfg]
    if c["kind"] == "tm":
        wl = tm_workload(wl_cfg, 0)
        U, V = wl["H"] - wl["h"] + 1, wl["W"] - wl["w"] + 1
        # size the per-step sample from a probe: ~ (target / steps) seconds of CPU work
        t0 = time.perf_counter()
        oracle.ncc_surface(wl["img"], wl["T"], 0, 1)
        per_row = time.perf_counter() - t0
        budget = max(0.5, 60.0 / max(1, args.steps + args.warmup))
        rows = int(max(1, min(U, budget / max(per_row, 1e-6))))
        times = []
        for s in range(args.warmup + args.steps):
            u0 = (s * rows) % max(1, U - rows + 1)
            t0 = time.perf_counter()
            oracle.ncc_surface(wl["img"], wl["T"], u0, u0 + rows)
            if s >= args.warmup:
                times.append(time.perf_counter() - t0)
        units = rows * V
        metric, unit = "NCC offsets/sec", "offsets/s"
        sample = f"{rows} offset rows x {V} cols of cfg{wl_cfg} ({units} offsets) per step"
    else:
        H, W, h, m, st = c["H"], c["W"], c["h"], c["m"], c["step"]
        dy, dx = synth.piv_shift_for_pair(wl_cfg, 0)
        p = synth.particle_pair_integer(H, W, dy, dx, seed=wl_cfg * 1000)
        Ky, Kx = oracle.piv_grid(H, W, h, h, m, m, st, st)
        t0 = time.perf_counter()
        oracle.piv_windows(p.A, p.B, h, h, m, m, st, st, [0], [0])
        per_win = time.perf_counter() - t0
        budget = max(0.5, 60.0 / max(1, args.steps + args.warmup))
        nwin = int(max(cores, min(Ky * Kx, budget * cores / max(per_win, 1e-6))))
        g = synth.rng(17)
        times = []
        for s in range(args.warmup + args.steps):
            kys, kxs = g.integers(0, Ky, nwin), g.integers(0, Kx, nwin)
            t0 = time.perf_counter()
            oracle.piv_windows(p.A, p.B, h, h, m, m, st, st, kys, kxs)
            if s >= args.warmup:
                times.append(time.perf_counter() - t0)
        units = nwin
        metric, unit = "PIV vectors/sec", "vectors/s"
        sample = f"{nwin} random windows of one cfg{wl_cfg} pair per step"
    tot = sum(times)
    value = units * len(times) / tot
    return dict(metric=metric, value=value, unit=unit, ms_per_step=1e3 * tot / len(times), sample=sample,
                cores=oracle.num_threads())


# ----------------------------------------------------------------------------- our arm
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--workload", default="cfg2", choices=["cfg1", "cfg2", "cfg3", "cfg4", "cfg5"])
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-secondary", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    args = ap.parse_args()
    args.warmup = max(3, args.warmup)
    cfg = int(args.workload[3:])
    ws, rank, local = dist_env()

    if args.impl == "reference":
        if rank != 0:
            return 0
        r = run_reference(args, cfg)
        line = {"metric": r["metric"], "value": r["value"], "unit": r["unit"], "n_gpus": args.gpus,
                "steps": args.steps, "warmup": args.warmup, "ms_per_step": r["ms_per_step"],
                "higher_is_better": True, "scaling": "strong" if cfg == 4 else "weak", "vs_baseline": None,
                "dtype": "f64",
                "data": "synthetic", "impl": "reference",
                "config": {"workload": f"cfg{cfg}", **{k: v for k, v in synth.CONFIGS[cfg].items()}},
                "cpu_baseline": {"value": r["value"], "unit": r["unit"], "cores": r["cores"], "kind": "oracle",
                                 "sample": r["sample"]},
                "e2e": {"value": r["value"], "unit": r["unit"], "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
        print(json.dumps(line), flush=True)
        return 0

    import torch
    import torch.distributed as dist
    from paper_conf_ipps_moorelk13_b200 import build as B
    from paper_conf_ipps_moorelk13_b200.api import MatchPlan, PivPlan, decode_peaks, decode_vectors

    if ws > 1:
        dist.init_process_group("nccl")
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if rank == 0:
        B.build()
    if ws > 1:
        dist.barrier()
    props = torch.cuda.get_device_properties(dev)
    sms = props.multi_processor_count
    flush = torch.empty(L2_FLUSH_BYTES // 4, dtype=torch.float32, device=dev)
    stream = torch.cuda.current_stream(dev)

    def run_steps(fn, n, plan=None):
        """n steps; per step: L2 flush (untimed), events around fn(); returns per-step ms and
        the numerator kernel ms reported by the plan's own events (same stream)."""
        step_ms, num_ms = [], []
        for _ in range(n):
            flush.zero_()
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            fn()
            e1.record(stream)
            e1.synchronize()
            step_ms.append(e0.elapsed_time(e1))
            if plan is not None:
                num_ms.append(plan.timing().numerator_ms)
        return step_ms, num_ms

    # cfg5 (BASELINE: "offset bands sharded across 8 GPUs"): under torchrun the one large match
    # is split into contiguous offset-row bands (strong scaling, same frame on every rank, peaks
    # merged with the tie rule); the other TM configs run one frame per rank (weak scaling)
    bands = cfg == 5 and ws > 1
    wl = (tm_workload(cfg, 0 if bands else rank) if synth.CONFIGS[cfg]["kind"] == "tm"
          else piv_workload(cfg, rank, ws))
    launches_per_step = 0
    if wl["kind"] == "tm":
        plan = MatchPlan(wl["H"], wl["W"], wl["h"], wl["w"], batch=1, device=local, timing=True,
                         shard_rank=rank if bands else 0, shard_count=ws if bands else 1)
        d_img = torch.from_numpy(wl["img"]).to(dev)
        d_t = torch.from_numpy(wl["T"]).to(dev)
        peaks = torch.empty((1, 4), dtype=torch.int32, device=dev)
        step = lambda: plan.match(d_img, d_t, stream=stream, peaks=peaks)  # noqa: E731
        units_per_step = plan.info.outputs_per_call
        metric, unit = "NCC offsets/sec", "offsets/s"
        launches_per_step = plan.info.launches_per_call
        h2d = wl["img"].nbytes + wl["T"].nbytes
        d2h = 16
        # host buffers for the end-to-end arm (pinned)
        h_img = torch.from_numpy(wl["img"]).pin_memory()
        h_t = torch.from_numpy(wl["T"]).pin_memory()
        h_pk = torch.empty((1, 4), dtype=torch.int32).pin_memory()
        e2e_step = lambda: plan.match_host(h_img, h_t, h_pk, stream=stream)  # noqa: E731
    else:
        plan = PivPlan(wl["H"], wl["W"], wl["h"], wl["m"], wl["step"], pairs=wl["pairs"], device=local, timing=True)
        A, Bf, shifts = piv_frames_device(wl, dev, torch)
        Ky, Kx = plan.grid
        vec = torch.empty((wl["pairs"], Ky, Kx, 6), dtype=torch.int32, device=dev)
        step = lambda: plan.correlate(A, Bf, stream=stream, vectors=vec)  # noqa: E731
        units_per_step = plan.info.outputs_per_call
        metric, unit = "PIV vectors/sec", "vectors/s"
        launches_per_step = plan.info.launches_per_call
        h2d = 2 * A.numel() * 4
        d2h = vec.numel() * 4
        # host frames (pinned); batches larger than one sub-batch stream through the plan's two
        # device slots (H2D of chunk c+1 overlapping the correlation of chunk c)
        hA = torch.empty(A.shape, dtype=A.dtype).pin_memory()
        hA.copy_(A)
        hB = torch.empty(Bf.shape, dtype=Bf.dtype).pin_memory()
        hB.copy_(Bf)
        hv = torch.empty(vec.shape, dtype=torch.int32).pin_memory()
        e2e_step = lambda: plan.correlate_host(hA, hB, hv, stream=stream)  # noqa: E731

    # ---- multi-GPU: every timed step ends with the path's only collective, the gather of the
    # 16-B peaks / 24-B vectors to all ranks (NCCL over NVLink, ordered on the compute stream)
    if ws > 1:
        res_t = peaks if wl["kind"] == "tm" else vec.reshape(-1, 6)
        gathered_t = torch.empty((ws,) + tuple(res_t.shape), dtype=res_t.dtype, device=dev)
        compute_step = step

        def step():
            compute_step()
            dist.all_gather_into_tensor(gathered_t, res_t)

    # ---- warmup, then the timed region (barrier + sync on both sides)
    run_steps(step, args.warmup, plan)
    sampler = ClockSampler(physical_gpu_index(local))
    sampler.start()
    time.sleep(0.3)
    if ws > 1:
        dist.barrier()
    torch.cuda.synchronize(dev)
    t_wall = time.perf_counter()
    step_ms, num_ms = run_steps(step, args.steps, plan)
    torch.cuda.synchronize(dev)
    if ws > 1:
        dist.barrier()
    t_wall = time.perf_counter() - t_wall
    clocks = sampler.stop()
    total_ms = sum(step_ms)

    # ---- result gather (the only collective: 16-B peaks / 24-B vectors over NCCL)
    if wl["kind"] == "tm":
        res = peaks.clone()
    else:
        res = vec.reshape(-1, 6)
    correct = None
    if wl["kind"] == "tm":
        pk = decode_peaks(peaks)
        correct = bool((int(pk["u"][0]), int(pk["v"][0])) == wl["planted"])
    else:
        d = decode_vectors(vec)
        want = torch.tensor(shifts, dtype=torch.int32, device=dev)
        correct = bool(((d["iy"] == want[:, 0, None, None]) & (d["ix"] == want[:, 1, None, None])).all())
    if ws > 1:
        gathered = torch.empty((ws,) + tuple(res.shape), dtype=res.dtype, device=dev)
        dist.all_gather_into_tensor(gathered, res.contiguous())
        if bands:  # the band peaks merged with the tie rule give the full match's peak
            from paper_conf_ipps_moorelk13_b200 import shard
            mk = decode_peaks(shard.merge_peaks(gathered.cpu(), plan.info.V))
            correct = bool((int(mk["u"][0]), int(mk["v"][0])) == wl["planted"])
        t = torch.tensor([total_ms], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        total_ms = float(t.item())
        ok = torch.tensor([1 if correct else 0], device=dev)
        dist.all_reduce(ok, op=dist.ReduceOp.MIN)
        correct = bool(ok.item())

    units_all = plan.info.U * plan.info.V if bands else units_per_step * ws  # whole-job units per step
    value = units_all * args.steps / (total_ms / 1e3)
    num_avg = sum(num_ms) / len(num_ms)
    flops = plan.info.flops_per_call
    achieved = flops / (num_avg / 1e3) / 1e12
    max_mhz = clocks.get("sm_max_mhz") or 1965.0
    sm_mhz = clocks.get("sm_mhz")
    tensor = plan.info.variant_name.decode().startswith("tm_tc")
    if tensor:
        # 3xTF32 on tcgen05: 3 tf32 MMAs per fp32 MAC.  tf32 peak = measured bf16 GEMM peak x the
        # nominal tf32/bf16 ratio (1.1 / 2.25 PFLOP/s, B200_PROFILING.md); the fp32-equivalent
        # peak of the method is a third of it.
        mp = {}
        try:
            mp = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
        except Exception:
            pass
        bf16 = mp.get("bf16_tflops") or 1590.0
        peak = bf16 * (1.1 / 2.25) / 3.0
        peak_note = (f"3xTF32 fp32-equivalent tensor peak = {'measured' if mp else 'fallback'} bf16 GEMM "
                     f"{bf16:.1f} TFLOP/s x (tf32/bf16 nominal 1.1/2.25) / 3 MMAs per MAC")
        peak_at_clock = peak * sm_mhz / max_mhz if sm_mhz else None
        # the hardware issue rate, from our own probe (tools/microbench/umma_probe.cu): a
        # cta_group::1 M=128 tf32 MMA of width N takes N/2 cycles (K=8) = 4096 tf32 FLOP/cycle/SM.
        # The cuBLAS-measured bf16 figure above is a power-capped GEMM and sits below it, so
        # frac can approach or pass 1 for a kernel running at full clock; this is the strict one.
        issue_peak = sms * 4096 * max_mhz * 1e6 / 3.0 / 1e12
        issue = {"issue_rate_peak": issue_peak, "frac_of_issue_rate": achieved / issue_peak,
                 "issue_rate_note": "SMs x 4096 tf32 FLOP/cycle (probe: N=136 MMA = 68 cycles) x max SM clock / 3"}
    else:
        issue = {}
        peak = sms * 128 * 2 * max_mhz * 1e6 / 1e12
        peak_note = "FP32 FFMA peak = SMs x 128 lanes x 2 FLOP x max SM clock (derived; MEASURED_PEAKS.json has no FP32 figure)"
        peak_at_clock = sms * 128 * 2 * sm_mhz * 1e6 / 1e12 if sm_mhz else None

    # ---- end-to-end through the host-buffer C-ABI call (H2D + compute + D2H in the region)
    e2e = None
    if e2e_step is not None:
        run_steps(e2e_step, 3)
        if ws > 1:
            dist.barrier()
        e_ms, _ = run_steps(e2e_step, args.steps)
        et = sum(e_ms)
        if ws > 1:
            t = torch.tensor([et], dtype=torch.float64, device=dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            et = float(t.item())
        e2e = {"value": units_all * args.steps / (et / 1e3), "unit": unit, "h2d_bytes_per_step": h2d,
               "d2h_bytes_per_step": d2h}

    # ---- traffic of the dominant kernel from the committed ncu capture (if present)
    traffic = None
    prof = os.path.join(ROOT, "profiles", "roofline_traffic.json")
    if os.path.exists(prof):
        try:
            tj = json.load(open(prof))
            traffic = tj.get(f"cfg{cfg}_tc" if tensor else f"cfg{cfg}")
            if traffic is None and f"cfg{cfg}_per_pair" in tj:
                traffic = tj[f"cfg{cfg}_per_pair"] * plan.info.grid_z
        except Exception:
            traffic = None

    line = {"metric": metric, "value": value, "unit": unit, "n_gpus": ws, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": total_ms / args.steps, "higher_is_better": True,
            "scaling": "strong" if (cfg == 4 or bands) else "weak", "vs_baseline": None, "dtype": "f32",
            "data": "synthetic",
            "config": {"workload": f"cfg{cfg}", **{k: v for k, v in synth.CONFIGS[cfg].items()},
                       "units_per_step_per_gpu": units_per_step, "l2": "flushed between steps (512 MiB write)",
                       "variant": plan.info.variant_name.decode(), "regs_per_thread": plan.info.regs_per_thread,
                       "parallelism": (f"bands{ws}" if bands else f"replicas{ws}") if wl["kind"] == "tm"
                       else f"pairs/{ws}"},
            "roofline": {"bound": "tensor" if tensor else "alu", "achieved": achieved, "peak": peak,
                         "unit": "TFLOP/s", "frac": achieved / peak, "traffic": traffic, "peak_note": peak_note,
                         "frac_at_sampled_clock": (achieved / peak_at_clock) if peak_at_clock else None,
                         "kernel_ms": num_avg, "kernel_share_of_step": num_avg / (total_ms / args.steps),
                         **issue},
            "clocks": clocks, "e2e": e2e, "gpu_launches": launches_per_step * args.steps,
            "correct": correct, "wall_s": t_wall}

    # ---- cpu baseline: the oracle on a bounded sample of the same workload (rank 0, N=1)
    if rank == 0 and ws == 1 and not args.no_cpu_baseline:
        class A_:  # noqa: N801
            steps, warmup = 1, 0
        try:
            r = run_reference(A_, cfg)
            line["cpu_baseline"] = {"value": r["value"], "unit": r["unit"], "cores": r["cores"], "kind": "oracle",
                                    "sample": r["sample"]}
        except Exception as e:  # pragma: no cover
            line["cpu_baseline"] = {"value": None, "unit": unit, "cores": cpu_cores(), "kind": "oracle",
                                    "sample": f"failed: {e}"}

    # ---- secondary: PIV cfg3 (one pair) on the same GPU, reported beside the headline
    if rank == 0 and ws == 1 and not args.no_secondary and cfg == 2:
        wl3 = piv_workload(3, 0, 1)
        p3 = PivPlan(wl3["H"], wl3["W"], wl3["h"], wl3["m"], wl3["step"], pairs=1, device=local, timing=True)
        A3, B3, sh3 = piv_frames_device(wl3, dev, torch)
        v3 = torch.empty((1,) + p3.grid + (6,), dtype=torch.int32, device=dev)
        st3 = lambda: p3.correlate(A3, B3, stream=stream, vectors=v3)  # noqa: E731
        run_steps(st3, 3, p3)
        s3, n3 = run_steps(st3, args.steps, p3)
        d3 = decode_vectors(v3)
        line["secondary"] = {"cfg3": {"metric": "PIV vectors/sec",
                                      "value": p3.info.outputs_per_call * len(s3) / (sum(s3) / 1e3),
                                      "ms_per_step": sum(s3) / len(s3),
                                      "numerator_tflops": p3.info.flops_per_call / (sum(n3) / len(n3) / 1e3) / 1e12,
                                      "variant": p3.info.variant_name.decode(),
                                      "correct": bool(((d3["iy"] == sh3[0][0]) & (d3["ix"] == sh3[0][1])).all())}}
        p3.close()

    if rank == 0:
        print(json.dumps(line), flush=True)
    plan.close()
    if ws > 1:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
