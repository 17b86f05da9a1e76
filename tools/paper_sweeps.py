#!/usr/bin/env python
"""Paper-shaped sweeps: structural analogues of the dissertation's
experiments whose numbers are lost (PAPER.md captions only):

  * Tab 6.13  TM partial sums, run-time evaluated (RE) vs specialised (SK) CUDA-core
                          kernels, beside the default tensor-core numerator (TC): time, TFLOP/s
                          and registers/thread.
  * Tab 6.4/6.16  PIV mask-size set   (masks 16..64, search +-16).
  * Tab 6.5/6.17  PIV search set  (mask 32, m = 4..32).
  * Tab 6.6/6.18  PIV overlap set (mask 32, m = 16, 0..75 % overlap).
  * Tab 5.2   the odd 156 x 116 template of Patient 4 (JIT specialised).

The paper's exact set members are lost with the text; the sets below keep their structure.
Every run is checked for correctness against the planted input (peak / displacement).
Prints one JSON object per line; python tools/paper_sweeps.py > out.jsonl
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_ipps_moorelk13_b200.api import MatchPlan, PivPlan, decode_peaks, decode_vectors  # noqa: E402

DEV = torch.device("cuda", 0)


def timed(plan, fn, reps=8):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    ns, tot = [], []
    for _ in range(reps):
        fn()
        t = plan.timing()
        ns.append(t.numerator_ms)
        tot.append(t.total_ms)
    return float(np.median(ns)), float(np.median(tot))


def emit(**kw):
    print(json.dumps(kw), flush=True)


def tm_re_vs_sk():
    for cfg in (2, 5):
        c = synth.CONFIGS[cfg]
        img, T, u0, v0 = synth.tm_inputs(cfg)
        d_img, d_t = torch.from_numpy(img).to(DEV), torch.from_numpy(T).to(DEV)
        for tier, generic, cc in (("TC", False, False), ("SK", False, True), ("RE", True, True)):
            with MatchPlan(c["H"], c["W"], c["h"], c["w"], timing=True, generic=generic, cuda_cores=cc) as plan:
                pk = None

                def run():
                    nonlocal pk
                    pk, _ = plan.match(d_img, d_t)
                num, tot = timed(plan, run, reps=8 if cfg == 2 else 3)
                d = decode_peaks(pk)
                emit(table="6.13", cfg=cfg, tier=tier, variant=plan.info.variant_name.decode(),
                     regs=plan.info.regs_per_thread, numerator_ms=num, step_ms=tot,
                     tflops=plan.info.flops_per_call / num / 1e9,
                     correct=(int(d["u"][0]), int(d["v"][0])) == (u0, v0))


def tm_odd_template():
    img = synth.uniform_image(1024, 1024, 52)
    T, u0, v0 = synth.planted_template(img, 156, 116, 53)
    d_img, d_t = torch.from_numpy(img).to(DEV), torch.from_numpy(T).to(DEV)
    for generic in (False, True):
        with MatchPlan(1024, 1024, 156, 116, timing=True, generic=generic) as plan:
            pk = None

            def run():
                nonlocal pk
                pk, _ = plan.match(d_img, d_t)
            num, tot = timed(plan, run)
            d = decode_peaks(pk)
            name = plan.info.variant_name.decode()
            emit(table="5.2", h=156, w=116, tier="RE" if generic else ("TC" if name.startswith("tm_tc") else "JIT"),
                 variant=name,
                 regs=plan.info.regs_per_thread, numerator_ms=num, step_ms=tot,
                 tflops=plan.info.flops_per_call / num / 1e9, correct=(int(d["u"][0]), int(d["v"][0])) == (u0, v0))


def piv_case(table, win, m, step, dy=5, dx=-3):
    p = synth.particle_pair_integer(1024, 1024, dy, dx, seed=900 + win + m + step)
    A = torch.from_numpy(p.A[None].copy()).to(DEV)
    B = torch.from_numpy(p.B[None].copy()).to(DEV)
    for generic in (False, True):
        with PivPlan(1024, 1024, win, m, step, pairs=1, timing=True, generic=generic) as plan:
            vec = None

            def run():
                nonlocal vec
                vec, _ = plan.correlate(A, B)
            num, tot = timed(plan, run)
            d = decode_vectors(vec)
            ok = bool(((d["iy"] == dy) & (d["ix"] == dx)).float().mean() > 0.99) if max(abs(dy), abs(dx)) < m else None
            emit(table=table, win=win, m=m, step=step, tier=["RE", "AOT", "JIT", "TC"][plan.info.specialized], variant=plan.info.variant_name.decode(),
                 regs=plan.info.regs_per_thread, vectors=plan.info.outputs_per_call, numerator_ms=num, step_ms=tot,
                 vectors_per_s=plan.info.outputs_per_call / (tot / 1e3),
                 tflops=plan.info.flops_per_call / num / 1e9, correct=ok)


def main():
    which = sys.argv[1:] or ["6.13", "5.2", "6.16", "6.17", "6.18"]
    if "6.13" in which:
        tm_re_vs_sk()
    if "5.2" in which:
        tm_odd_template()
    if "6.16" in which:
        for win in (16, 24, 32, 48, 64):
            piv_case("6.16", win, 16, win // 2)
    if "6.17" in which:
        for m in (4, 8, 12, 16, 24, 32):
            piv_case("6.17", 32, m, 16, dy=min(3, m - 1), dx=-min(2, m - 1))
    if "6.18" in which:
        for step in (32, 24, 16, 8):
            piv_case("6.18", 32, 16, step)


if __name__ == "__main__":
    main()
