#!/usr/bin/env python
"""Benchmark of the B200 NCC hot path (BASELINE.json metric: NCC offsets/s & PIV vectors/s at
1/2/4/8 B200, % of the FP32 roofline).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--workload cfg2|cfg1|cfg3|cfg4|cfg5]
                    [--impl ours|reference] [--no-secondary] [--no-cpu-baseline] [--backend nccl|gloo]

A step is one pass of the whole hot path over one batch of synthetic input: for TM
(cfg1/2/5) template prep -> fp64 window sums -> numerator -> normalise/argmax -> peak
(SURVEY.md 8(a) a1-a5); for PIV (cfg3/4) window sums -> batched correlation + peak +
sub-pixel (a2, a6, a7).  Default workload = configs[1] (cfg2: 128x128 template in a
1024x1024 image, 804,609 offsets).  At N = 1 the line also carries secondary objects for
cfg3, cfg4 and cfg5 (each with its own roofline, e2e, cpu_baseline and clocks; cfg4 = the
whole 256-pair batch on one GPU).  N > 1 (torchrun, one rank per GPU): cfg1-3 weak scaling
(every rank its own frame / pair), cfg4 the 256 pairs split across ranks, cfg5 the one
4096^2 match split into offset-row bands; every timed step ends with the path's only
collective, the all-gather of the 16-B peaks / 24-B vectors (NCCL over NVLink; --backend gloo
is a dry run of the same branch on one GPU).

--impl reference times the fp64 CPU oracle (oracle/, the only reference that exists for
this paper) on a bounded sample of the same workload, on rank 0 only.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
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
    """SM clock + throttle reasons sampled through NVML every ~1 ms on a background thread;
    only samples taken while `inside` is set (the timed region) are reported."""
    REASONS = {0x8: "hw_slowdown", 0x40: "hw_thermal_slowdown", 0x20: "sw_thermal_slowdown",
               0x4: "sw_power_cap"}

    def __init__(self, gpu):
        self.gpu = int(gpu) if str(gpu).isdigit() else 0
        self.rows, self.inside, self.stop_ev = [], False, threading.Event()
        self.h = None
        self.max_mhz = None

    def start(self):
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(self.gpu)
            self.max_mhz = float(pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM))
        except Exception:
            self.h = None
            return
        self.th = threading.Thread(target=self._run, daemon=True)
        self.th.start()

    def _run(self):
        nv = self.nv
        while not self.stop_ev.is_set():
            if self.inside:
                try:
                    mhz = nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM)
                    rs = nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                    self.rows.append((float(mhz), int(rs)))
                except Exception:
                    pass
            time.sleep(0.001)

    def stop(self):
        if self.h is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"], "samples": 0}
        self.stop_ev.set()
        self.th.join(timeout=2)
        sm = [r[0] for r in self.rows]
        reasons = sorted({name for _, rs in self.rows for bit, name in self.REASONS.items() if rs & bit})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": self.max_mhz, "reasons": reasons,
                "samples": len(sm), "how": "NVML every ~1 ms, only inside the timed region"}


def cpu_cores():
    try:
        return len(os.sched_getaffinity(0))
    except Exception:
        return os.cpu_count() or 1


def cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except Exception:
        pass
    return "unknown"


def measured_peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        return {}


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
def run_reference(cfg, steps, warmup, budget_s, threads=None):
    """fp64 CPU oracle timed on this host, a bounded sample per step (~budget_s of CPU work
    per step).  threads=None: every core of the process's affinity mask."""
    import oracle
    cores = cpu_cores()
    oracle.set_num_threads(threads or cores)
    c = synth.CONFIGS[cfg]
    if c["kind"] == "tm":
        wl = tm_workload(cfg, 0)
        U, V = wl["H"] - wl["h"] + 1, wl["W"] - wl["w"] + 1
        t0 = time.perf_counter()
        oracle.ncc_surface(wl["img"], wl["T"], 0, 1)
        per_row = time.perf_counter() - t0
        rows = int(max(1, min(U, budget_s / max(per_row, 1e-6))))
        if rows > 1:  # refine with a multi-row probe (one row underuses the threads)
            k = min(rows, max(1, oracle.num_threads()))
            t0 = time.perf_counter()
            oracle.ncc_surface(wl["img"], wl["T"], 0, k)
            rows = int(max(1, min(U, budget_s * k / max(time.perf_counter() - t0, 1e-6))))
        times = []
        for s in range(warmup + steps):
            u0 = (s * rows) % max(1, U - rows + 1)
            t0 = time.perf_counter()
            oracle.ncc_surface(wl["img"], wl["T"], u0, u0 + rows)
            if s >= warmup:
                times.append(time.perf_counter() - t0)
        units = rows * V
        metric, unit = "NCC offsets/sec", "offsets/s"
        sample = f"{rows} offset rows x {V} cols of cfg{cfg} ({units} offsets) per step"
    else:
        H, W, h, m, st = c["H"], c["W"], c["h"], c["m"], c["step"]
        dy, dx = synth.piv_shift_for_pair(cfg, 0)
        p = synth.particle_pair_integer(H, W, dy, dx, seed=cfg * 1000)
        Ky, Kx = oracle.piv_grid(H, W, h, h, m, m, st, st)
        nth = max(1, oracle.num_threads())
        t0 = time.perf_counter()
        oracle.piv_windows(p.A, p.B, h, h, m, m, st, st, [0] * nth, [0] * nth)
        per_round = time.perf_counter() - t0
        nwin = int(max(nth, min(Ky * Kx, budget_s * nth / max(per_round, 1e-6))))
        g = synth.rng(17)
        times = []
        for s in range(warmup + steps):
            kys, kxs = g.integers(0, Ky, nwin), g.integers(0, Kx, nwin)
            t0 = time.perf_counter()
            oracle.piv_windows(p.A, p.B, h, h, m, m, st, st, kys, kxs)
            if s >= warmup:
                times.append(time.perf_counter() - t0)
        units = nwin
        metric, unit = "PIV vectors/sec", "vectors/s"
        sample = f"{nwin} random windows of one cfg{cfg} pair per step"
    tot = sum(times)
    used = oracle.num_threads()
    oracle.set_num_threads(cores)
    return dict(metric=metric, value=units * len(times) / tot, unit=unit, ms_per_step=1e3 * tot / len(times),
                sample=sample, cores=used)


def cpu_baseline(cfg, budget_s):
    """The oracle on all host cores AND on one thread, with the CPU model."""
    r = run_reference(cfg, 1, 0, budget_s)
    r1 = run_reference(cfg, 1, 0, max(0.5, budget_s / 4), threads=1)
    return {"value": r["value"], "unit": r["unit"], "cores": r["cores"], "kind": "oracle", "sample": r["sample"],
            "value_1thread": r1["value"], "sample_1thread": r1["sample"], "cpu_model": cpu_model()}


# ----------------------------------------------------------------------------- our arm
class Ctx:
    pass


def run_steps(ctx, fn, n, plan=None):
    """n steps; per step: L2 flush (untimed), CUDA events on the launching stream around fn();
    returns per-step ms and the numerator kernel ms from the plan's own events (same stream)."""
    torch = ctx.torch
    step_ms, num_ms = [], []
    for _ in range(n):
        ctx.flush.zero_()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(ctx.stream)
        fn()
        e1.record(ctx.stream)
        e1.synchronize()
        step_ms.append(e0.elapsed_time(e1))
        if plan is not None:
            num_ms.append(plan.timing().numerator_ms)
    return step_ms, num_ms


def max_over_ranks(ctx, x):
    if ctx.ws == 1:
        return x
    torch, dist = ctx.torch, ctx.dist
    t = torch.tensor([x], dtype=torch.float64, device=ctx.coll_dev)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def roofline(ctx, plan, flops, num_avg, step_ms, clocks, cfg, pairs=None):
    """Roofline object of the dominant (numerator) kernel."""
    sms = ctx.sms
    achieved = flops / (num_avg / 1e3) / 1e12
    max_mhz = clocks.get("sm_max_mhz") or 1965.0
    sm_mhz = clocks.get("sm_mhz")
    fp32_peak = sms * 128 * 2 * max_mhz * 1e6 / 1e12
    vname = plan.info.variant_name.decode()
    tensor = vname.startswith(("tm_tc", "piv_tc"))
    kname = ("tm_tc_kernel" if vname.startswith("tm_tc") else
             "piv_tc_kernel + piv_tc_border_kernel (numerator: tensor cores + its last column)"
             if vname.startswith("piv_tc") else vname)
    extra = {"fp32_peak": fp32_peak, "frac_of_fp32_peak": achieved / fp32_peak,
             "fp32_peak_note": "SMs x 128 FP32 lanes x 2 FLOP x max SM clock (B200_PROFILING.md unit counts)"}
    if tensor:
        mp = measured_peaks()
        bf16 = mp.get("bf16_tflops") or 1590.0
        if vname.startswith(("piv_tc", "tm_tc_bf16")):
            # 3xBF16 on tcgen05 (kind::f16): 3 bf16 MMAs per fp32-equivalent MAC
            peak = bf16 / 3.0
            peak_note = (f"3xBF16 fp32-equivalent tensor peak = {'measured' if mp else 'fallback'} bf16 GEMM "
                         f"{bf16:.1f} TFLOP/s / 3 MMAs per MAC")
            issue_peak = sms * 8192 * max_mhz * 1e6 / 3.0 / 1e12
            issue_note = ("SMs x 8192 bf16 FLOP/cycle (probe: an M=128 K=16 MMA of width N takes N/2 cycles when "
                          "issued back to back, tools/microbench/issue_probe.cu) x max SM clock / 3")
        else:
            # 3xTF32 on tcgen05: 3 tf32 MMAs per fp32 MAC.  tf32 peak = measured bf16 GEMM peak x the
            # nominal tf32/bf16 ratio (1.1 / 2.25 PFLOP/s); the fp32-equivalent peak is a third of it.
            peak = bf16 * (1.1 / 2.25) / 3.0
            peak_note = (f"3xTF32 fp32-equivalent tensor peak = {'measured' if mp else 'fallback'} bf16 GEMM "
                         f"{bf16:.1f} TFLOP/s x (tf32/bf16 nominal 1.1/2.25) / 3 MMAs per MAC")
            # our own issue-rate probe (tools/microbench/umma_probe.cu): a cta_group::1 M=128 tf32
            # MMA of width N takes N/2 cycles (K=8) = 4096 tf32 FLOP/cycle/SM -- the strict one
            issue_peak = sms * 4096 * max_mhz * 1e6 / 3.0 / 1e12
            issue_note = "SMs x 4096 tf32 FLOP/cycle (probe: N=136 MMA = 68 cycles) x max SM clock / 3"
        peak_at_clock = peak * sm_mhz / max_mhz if sm_mhz else None
        extra.update({"issue_rate_peak": issue_peak, "frac_of_issue_rate": achieved / issue_peak,
                      "issue_rate_note": issue_note})
        bound = "tensor"
    else:
        peak = fp32_peak
        peak_note = "FP32 FFMA peak (derived; MEASURED_PEAKS.json has no FP32 figure)"
        peak_at_clock = sms * 128 * 2 * sm_mhz * 1e6 / 1e12 if sm_mhz else None
        bound = "alu"
    traffic = None
    prof = os.path.join(ROOT, "profiles", "roofline_traffic.json")
    if os.path.exists(prof):
        try:
            tj = json.load(open(prof))
            traffic = tj.get(f"cfg{cfg}_tc" if tensor else f"cfg{cfg}")
            pp = f"cfg{cfg}_tc_per_pair" if tensor else f"cfg{cfg}_per_pair"
            if traffic is None and pp in tj and pairs:  # per call, like `achieved`
                traffic = tj[pp] * pairs
        except Exception:
            traffic = None
    return {"bound": bound, "achieved": achieved, "peak": peak, "unit": "TFLOP/s", "frac": achieved / peak,
            "traffic": traffic, "peak_note": peak_note,
            "frac_at_sampled_clock": (achieved / peak_at_clock) if peak_at_clock else None,
            "kernel": kname,
            "kernel_ms": num_avg, "kernel_share_of_step": num_avg / step_ms, **extra}


def measure(ctx, cfg, steps, warmup, headline=True, cpu_budget=10.0):
    """One workload end to end: device-resident timed steps, roofline, e2e, clocks (and the
    oracle cpu_baseline on rank 0 at N=1).  Returns the JSON object."""
    torch, ws, rank, local, dev, stream = ctx.torch, ctx.ws, ctx.rank, ctx.local, ctx.dev, ctx.stream
    from paper_conf_ipps_moorelk13_b200.api import MatchPlan, PivPlan, decode_peaks, decode_vectors
    dist = ctx.dist
    multi = ws > 1 and headline
    bands = cfg == 5 and multi
    kind = synth.CONFIGS[cfg]["kind"]
    wl = tm_workload(cfg, 0 if bands else rank) if kind == "tm" else piv_workload(cfg, rank, ws if multi else 1)
    if kind == "tm":
        plan = MatchPlan(wl["H"], wl["W"], wl["h"], wl["w"], batch=1, device=local, timing=True,
                         shard_rank=rank if bands else 0, shard_count=ws if bands else 1)
        d_img = torch.from_numpy(wl["img"]).to(dev)
        d_t = torch.from_numpy(wl["T"]).to(dev)
        peaks = torch.empty((1, 4), dtype=torch.int32, device=dev)
        step = lambda: plan.match(d_img, d_t, stream=stream, peaks=peaks)  # noqa: E731
        metric, unit = "NCC offsets/sec", "offsets/s"
        frames_per_step = 1
        h2d = wl["img"].nbytes + wl["T"].nbytes
        d2h = 16
        h_img = torch.from_numpy(wl["img"]).pin_memory()
        h_t = torch.from_numpy(wl["T"]).pin_memory()
        h_pk = torch.empty((1, 4), dtype=torch.int32).pin_memory()
        e2e_step = lambda: plan.match_host(h_img, h_t, h_pk, stream=stream)  # noqa: E731
        res_t = peaks
    else:
        plan = PivPlan(wl["H"], wl["W"], wl["h"], wl["m"], wl["step"], pairs=wl["pairs"], device=local, timing=True)
        A, Bf, shifts = piv_frames_device(wl, dev, torch)
        Ky, Kx = plan.grid
        vec = torch.empty((wl["pairs"], Ky, Kx, 6), dtype=torch.int32, device=dev)
        step = lambda: plan.correlate(A, Bf, stream=stream, vectors=vec)  # noqa: E731
        metric, unit = "PIV vectors/sec", "vectors/s"
        frames_per_step = wl["pairs"]
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
        res_t = vec.reshape(-1, 6)
    units_per_step = plan.info.outputs_per_call
    launches_per_step = plan.info.launches_per_call

    # multi-GPU: every timed step ends with the path's only collective, the gather of the 16-B
    # peaks / 24-B vectors (NCCL over NVLink; gloo dry run: through the host)
    if multi:
        from paper_conf_ipps_moorelk13_b200 import shard
        compute_step = step
        if ctx.backend == "nccl":
            gathered_t = torch.empty((ws,) + tuple(res_t.shape), dtype=res_t.dtype, device=dev)

            def step():
                compute_step()
                dist.all_gather_into_tensor(gathered_t, res_t)
        else:
            def step():
                compute_step()
                shard.gather_results(res_t)

    run_steps(ctx, step, warmup, plan)
    sampler = ClockSampler(physical_gpu_index(local))
    sampler.start()
    if multi:
        dist.barrier()
    torch.cuda.synchronize(dev)
    sampler.inside = True
    t_wall = time.perf_counter()
    step_ms, num_ms = run_steps(ctx, step, steps, plan)
    torch.cuda.synchronize(dev)
    t_wall = time.perf_counter() - t_wall
    sampler.inside = False
    if multi:
        dist.barrier()
    clocks = sampler.stop()
    total_ms = max_over_ranks(ctx, sum(step_ms)) if multi else sum(step_ms)

    # correctness of the timed result (planted peak / shifts), merged over ranks
    if kind == "tm":
        pk = decode_peaks(peaks)
        correct = bool((int(pk["u"][0]), int(pk["v"][0])) == wl["planted"])
    else:
        d = decode_vectors(vec)
        want = torch.tensor(shifts, dtype=torch.int32, device=dev)
        correct = bool(((d["iy"] == want[:, 0, None, None]) & (d["ix"] == want[:, 1, None, None])).all())
    if multi:
        from paper_conf_ipps_moorelk13_b200 import shard
        gathered = shard.gather_results(res_t.clone())
        if bands:  # the band peaks merged with the tie rule give the full match's peak (on device)
            mk = decode_peaks(shard.merge_peaks(gathered, plan.info.V))
            correct = bool((int(mk["u"][0]), int(mk["v"][0])) == wl["planted"])
        correct = max_over_ranks(ctx, 0.0 if correct else 1.0) == 0.0

    units_all = plan.info.U * plan.info.V if bands else units_per_step * (ws if multi else 1)
    frames_all = 1 if bands else frames_per_step * (ws if multi else 1)
    sec = total_ms / 1e3
    value = units_all * steps / sec
    num_avg = sum(num_ms) / len(num_ms)
    rl = roofline(ctx, plan, plan.info.flops_per_call, num_avg, total_ms / steps, clocks, cfg,
                  pairs=wl.get("pairs") if kind == "piv" else None)
    tensor = rl["bound"] == "tensor"

    # end to end through the host-buffer C-ABI call (H2D + compute + D2H in the region)
    run_steps(ctx, e2e_step, 3)
    if multi:
        dist.barrier()
    e_ms, _ = run_steps(ctx, e2e_step, steps)
    et = max_over_ranks(ctx, sum(e_ms)) if multi else sum(e_ms)
    e2e = {"value": units_all * steps / (et / 1e3), "unit": unit, "h2d_bytes_per_step": h2d,
           "d2h_bytes_per_step": d2h, "ms_per_step": et / steps,
           "api": "ncc_match_host" if kind == "tm" else "piv_correlate_host"}
    if kind == "tm" and not multi:
        # a stream of frames through the same public call: 8 frames per call, the host->device
        # copy of the next chunk overlapping the match of the current one, beside the
        # device-resident rate of the same 8-frame batch
        F = 8
        p8 = MatchPlan(wl["H"], wl["W"], wl["h"], wl["w"], batch=F, device=local)
        hs = torch.from_numpy(np.ascontiguousarray(np.broadcast_to(wl["img"], (F,) + wl["img"].shape))).pin_memory()
        hp8 = torch.empty((F, 4), dtype=torch.int32).pin_memory()
        ds = hs.to(dev)
        dp8 = torch.empty((F, 4), dtype=torch.int32, device=dev)
        st8 = min(steps, 10)
        run_steps(ctx, lambda: p8.match_host(hs, h_t, hp8, stream=stream), 3)
        s_ms, _ = run_steps(ctx, lambda: p8.match_host(hs, h_t, hp8, stream=stream), st8)
        run_steps(ctx, lambda: p8.match(ds, d_t, stream=stream, peaks=dp8), 3)
        d_ms, _ = run_steps(ctx, lambda: p8.match(ds, d_t, stream=stream, peaks=dp8), st8)
        u8 = p8.info.outputs_per_call
        ok8 = bool((decode_peaks(hp8)["u"] == wl["planted"][0]).all() and (decode_peaks(hp8)["v"] == wl["planted"][1]).all())
        e2e["stream8"] = {"value": u8 * st8 / (sum(s_ms) / 1e3), "unit": unit, "frames_per_call": F,
                          "h2d_bytes_per_step": F * wl["img"].nbytes + wl["T"].nbytes,
                          "d2h_bytes_per_step": F * 16, "ms_per_step": sum(s_ms) / st8,
                          "device_value_same_batch": u8 * st8 / (sum(d_ms) / 1e3),
                          "frac_of_device_same_batch": sum(d_ms) / sum(s_ms), "correct": ok8}
        p8.close()
        del hs, ds

    c = synth.CONFIGS[cfg]
    line = {"metric": metric, "value": value, "unit": unit, "n_gpus": ws if multi else 1, "steps": steps,
            "warmup": warmup, "ms_per_step": total_ms / steps, "higher_is_better": True,
            "scaling": "strong" if (multi and (cfg == 4 or bands)) else "weak", "vs_baseline": None,
            "dtype": "bf16x3" if tensor else "f32",
            "arith": ("3xBF16 on tcgen05 tensor cores (kind::f16, fp32-emulated: hi*hi + hi*lo + lo*hi with "
                      "hi = bf16(x), lo = bf16(x - hi), fp32 accumulate)" +
                      ("; last output column on FFMA" if rl["kernel"].startswith("piv_tc") else
                       "; ragged last columns on FFMA") + "; fp64 window sums, fp64 variance") if tensor else
                     "fp32 FFMA numerator; fp64 window sums, fp64 variance",
            "data": "synthetic",
            "frames_per_s" if kind == "tm" else "pairs_per_s": frames_all * steps / sec,
            "config": {"workload": f"cfg{cfg}", **{k: v for k, v in c.items()},
                       "units_per_step_per_gpu": units_per_step,
                       "l2": "flushed between steps (512 MiB write)",
                       "variant": plan.info.variant_name.decode(), "regs_per_thread": plan.info.regs_per_thread,
                       "parallelism": ((f"bands{ws}" if bands else f"replicas{ws}") if kind == "tm"
                                       else f"pairs/{ws}") if multi else "1gpu"},
            "roofline": rl, "clocks": clocks, "e2e": e2e, "gpu_launches": launches_per_step * steps,
            "correct": correct, "wall_s": t_wall}
    if rank == 0 and not multi and not ctx.no_cpu:
        try:
            line["cpu_baseline"] = cpu_baseline(cfg, cpu_budget)
        except Exception as e:  # pragma: no cover
            line["cpu_baseline"] = {"value": None, "unit": unit, "cores": cpu_cores(), "kind": "oracle",
                                    "sample": f"failed: {e}"}
    plan.close()
    return line


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--workload", default="cfg2", choices=["cfg1", "cfg2", "cfg3", "cfg4", "cfg5"])
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-secondary", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--backend", default="nccl", choices=["nccl", "gloo"],
                    help="process-group backend under torchrun (gloo: dry run of the multi-GPU branch)")
    args = ap.parse_args()
    args.warmup = max(3, args.warmup)
    cfg = int(args.workload[3:])
    ws, rank, local = dist_env()

    if args.impl == "reference":
        if rank != 0:
            return 0
        budget = max(0.5, 60.0 / max(1, args.steps + args.warmup))
        r = run_reference(cfg, args.steps, args.warmup, budget)
        line = {"metric": r["metric"], "value": r["value"], "unit": r["unit"], "n_gpus": args.gpus,
                "steps": args.steps, "warmup": args.warmup, "ms_per_step": r["ms_per_step"],
                "higher_is_better": True, "scaling": "strong" if cfg == 4 else "weak", "vs_baseline": None,
                "dtype": "f64", "data": "synthetic", "impl": "reference",
                "config": {"workload": f"cfg{cfg}", **{k: v for k, v in synth.CONFIGS[cfg].items()}},
                "cpu_baseline": {"value": r["value"], "unit": r["unit"], "cores": r["cores"], "kind": "oracle",
                                 "sample": r["sample"], "cpu_model": cpu_model()},
                "e2e": {"value": r["value"], "unit": r["unit"], "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
        print(json.dumps(line), flush=True)
        return 0

    import torch
    import torch.distributed as dist
    from paper_conf_ipps_moorelk13_b200 import build as B

    if args.backend == "gloo":  # dry run: ranks may share the GPUs there are
        local = local % max(1, torch.cuda.device_count())
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if ws > 1:
        if args.backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group("gloo")
    if rank == 0:
        B.build()
    if ws > 1:
        dist.barrier()
    ctx = Ctx()
    ctx.torch, ctx.dist, ctx.ws, ctx.rank, ctx.local, ctx.dev = torch, dist, ws, rank, local, dev
    ctx.backend = args.backend
    ctx.coll_dev = dev if args.backend == "nccl" else torch.device("cpu")
    ctx.sms = torch.cuda.get_device_properties(dev).multi_processor_count
    ctx.flush = torch.empty(L2_FLUSH_BYTES // 4, dtype=torch.float32, device=dev)
    ctx.stream = torch.cuda.current_stream(dev)
    ctx.no_cpu = args.no_cpu_baseline

    line = measure(ctx, cfg, args.steps, args.warmup, headline=True, cpu_budget=20.0)

    # secondary workloads on the same GPU (N = 1 only): every other config the metric names,
    # each with its own roofline / e2e / cpu_baseline / clocks
    if rank == 0 and ws == 1 and not args.no_secondary:
        sec = {}
        for c2 in (3, 4, 5):
            if c2 == cfg:
                continue
            st = min(args.steps, 10) if c2 == 4 else args.steps
            try:
                sec[f"cfg{c2}"] = measure(ctx, c2, st, args.warmup, headline=False, cpu_budget=8.0)
            except Exception as e:  # pragma: no cover
                sec[f"cfg{c2}"] = {"error": repr(e)}
            torch.cuda.empty_cache()
        line["secondary"] = sec

    if rank == 0:
        print(json.dumps(line), flush=True)
    if ws > 1:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
