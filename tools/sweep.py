#!/usr/bin/env python
"""Variant / split sweep on the GPU (paper Tab 6.13 / 6.21 analogue: % of best vs tile shape).

  python tools/sweep.py tm 2            # all TM variants valid for cfg2 x splits
  python tools/sweep.py piv 4 [pairs]   # PIV variants for cfg4
Prints one JSON line per (variant, split) with the numerator TFLOP/s from the plan's events.
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_ipps_moorelk13_b200.api import MatchPlan, PivPlan  # noqa: E402


def time_plan(plan, fn, reps=10):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    ms = []
    for _ in range(reps):
        fn()
        ms.append(plan.timing().numerator_ms)
    return float(np.median(ms))


def tm(cfg, variants, splits):
    c = synth.CONFIGS[cfg]
    img, T, _, _ = synth.tm_inputs(cfg)
    dev = torch.device("cuda", 0)
    d_img, d_t = torch.from_numpy(img).to(dev), torch.from_numpy(T).to(dev)
    for v in variants:
        for s in splits:
            if v:
                os.environ["NCC_FORCE_VARIANT"] = v
            else:
                os.environ.pop("NCC_FORCE_VARIANT", None)
            if s:
                os.environ["NCC_FORCE_SPLIT"] = str(s)
            else:
                os.environ.pop("NCC_FORCE_SPLIT", None)
            with MatchPlan(c["H"], c["W"], c["h"], c["w"], timing=True) as plan:
                ms = time_plan(plan, lambda: plan.match(d_img, d_t))
                print(json.dumps({"cfg": cfg, "variant": plan.info.variant_name.decode(), "ms": ms,
                                  "tflops": plan.info.flops_per_call / ms / 1e9,
                                  "regs": plan.info.regs_per_thread, "smem": plan.info.smem_per_block,
                                  "grid": plan.info.grid_x}), flush=True)


if __name__ == "__main__" and sys.argv[1] == "tm":
    kind, cfg = sys.argv[1], int(sys.argv[2])
    if kind == "tm":
        vs = [None, "tm_sk_128x128_rv12_lx4_8x1_c32x64", "tm_sk_128x128_rv12_lx4_4x2_c32x64",
              "tm_sk_128x128_rv12_lx4_4x1_c16x64", "tm_sk_128x128_rv12_lx4_8x1_c16x64"] if cfg == 2 else [None]
        for ct in (None,):
            if ct:
                os.environ["NCC_NO_CONST_TPL"] = ct
            else:
                os.environ.pop("NCC_NO_CONST_TPL", None)
            tm(cfg, vs, [None, 1, 2, 4, 6, 8, 12, 16] if cfg == 2 else [None])


def piv(cfg, variants, pairs):
    import bench
    c = synth.CONFIGS[cfg]
    wl = dict(cfg=cfg, H=c["H"], W=c["W"], h=c["h"], w=c["w"], m=c["m"], step=c["step"], pairs=pairs, rank=0)
    dev = torch.device("cuda", 0)
    A, B, _ = bench.piv_frames_device(wl, dev, torch)
    for v in variants:
        if v:
            os.environ["NCC_FORCE_VARIANT"] = v
        else:
            os.environ.pop("NCC_FORCE_VARIANT", None)
        with PivPlan(c["H"], c["W"], c["h"], c["m"], c["step"], pairs=pairs, timing=True) as plan:
            ms = time_plan(plan, lambda: plan.correlate(A, B), reps=5)
            print(json.dumps({"cfg": cfg, "variant": plan.info.variant_name.decode(), "ms": ms,
                              "tflops": plan.info.flops_per_call / ms / 1e9, "regs": plan.info.regs_per_thread,
                              "smem": plan.info.smem_per_block, "grid": plan.info.grid_x}), flush=True)


if __name__ == "__main__" and sys.argv[1] == "piv":
    cfg = int(sys.argv[2])
    vs = {3: [None, "piv_sk_32x32_m16_rv12_nt512_w5", "piv_sk_32x32_m16_rv12_nt512_w4", "piv_re_rv12_cw16_nt256"],
          4: [None, "piv_sk_64x64_m32_rv12_nt512_w1", "piv_re_rv12_cw16_nt256"]}[cfg]
    piv(cfg, vs, 1 if cfg == 3 else 16)
