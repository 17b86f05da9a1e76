#!/usr/bin/env python
"""Sensitivity surfaces: the dissertation's Tab 6.21 / 6.22 analogues,
"% of peak performance" over a grid of kernel configurations (captions only):

  * Tab 6.21 (TM): main tile size x threads per block, run-time specialised (NVRTC)
    CUDA-core numerator kernels on the cfg2 problem (1024^2 image, 128^2 template): tile =
    (8 WY) output rows x (4 RV WX) output columns, threads = 32 WX WY (NCC_TM_JIT).
  * Tab 6.22 (PIV): data registers (offsets per thread, RV) x threads per block, the
    run-time specialised PIV kernel on the cfg3 problem (1024^2 pair, 32^2 masks, +-16, step 16):
    threads = WPB windows x ceil(items / 32) warps (NCC_PIV_JIT).

Each point is checked against its planted input; % of best is relative to the fastest point of
its table.  Prints one JSON object per line: python tools/sensitivity.py > out.jsonl
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


def timed(plan, fn, reps=10):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    ms = []
    for _ in range(reps):
        fn()
        ms.append(plan.timing().numerator_ms)
    return float(np.median(ms))


def emit(**kw):
    print(json.dumps(kw), flush=True)


def tm_surface():
    c = synth.CONFIGS[2]
    img, T, u0, v0 = synth.tm_inputs(2)
    d_img, d_t = torch.from_numpy(img).to(DEV), torch.from_numpy(T).to(DEV)
    for RV in (4, 8, 12, 16):
        for WX, WY in ((1, 1), (1, 2), (2, 1), (1, 4), (2, 2), (4, 1), (1, 8), (2, 4), (4, 2)):
            BU, BV = 8 * WY, 4 * RV * WX
            if BV + 64 > 256:  # TMA box width limit (staged columns = BV + CW)
                continue
            os.environ["NCC_TM_JIT"] = f"{RV},4,{WX},{WY},16,64"
            try:
                with MatchPlan(c["H"], c["W"], c["h"], c["w"], timing=True, cuda_cores=True) as plan:
                    name = plan.info.variant_name.decode()
                    if not name.startswith("tm_jit"):
                        emit(table="6.21", RV=RV, WX=WX, WY=WY, error="not specialised: " + name)
                        continue
                    pk = None

                    def run():
                        nonlocal pk
                        pk, _ = plan.match(d_img, d_t)
                    ms = timed(plan, run)
                    d = decode_peaks(pk)
                    ok = (int(d["u"][0]), int(d["v"][0])) == (u0, v0)
                    emit(table="6.21", RV=RV, WX=WX, WY=WY, tile_rows=BU, tile_cols=BV, tile=BU * BV,
                         threads=32 * WX * WY, regs=plan.info.regs_per_thread, variant=name, numerator_ms=ms,
                         tflops=plan.info.flops_per_call / ms / 1e9, correct=ok)
            except Exception as e:  # a configuration the device cannot run (resources)
                emit(table="6.21", RV=RV, WX=WX, WY=WY, error=repr(e)[:160])
    os.environ.pop("NCC_TM_JIT", None)


def piv_surface():
    c = synth.CONFIGS[3]
    dy, dx = synth.piv_shift_for_pair(3, 0)
    p = synth.particle_pair_integer(c["H"], c["W"], dy, dx, seed=3000)
    A = torch.from_numpy(p.A[None].copy()).to(DEV)
    B = torch.from_numpy(p.B[None].copy()).to(DEV)
    for RV in (4, 8, 12, 16, 20, 24):
        for WPB in (1, 2, 3, 4):
            os.environ["NCC_PIV_JIT"] = f"{RV},{WPB}"
            try:
                with PivPlan(c["H"], c["W"], c["h"], c["m"], c["step"], pairs=1, timing=True) as plan:
                    name = plan.info.variant_name.decode()
                    if not name.startswith("piv_jit"):
                        emit(table="6.22", RV=RV, WPB=WPB, error="not specialised: " + name)
                        continue
                    vec = None

                    def run():
                        nonlocal vec
                        vec, _ = plan.correlate(A, B)
                    ms = timed(plan, run)
                    d = decode_vectors(vec)
                    ok = bool(((d["iy"] == dy) & (d["ix"] == dx)).all())
                    emit(table="6.22", RV=RV, WPB=WPB, threads=plan.info.threads_per_block,
                         regs=plan.info.regs_per_thread, smem=plan.info.smem_per_block, variant=name,
                         numerator_ms=ms, tflops=plan.info.flops_per_call / ms / 1e9, correct=ok)
            except Exception as e:
                emit(table="6.22", RV=RV, WPB=WPB, error=repr(e)[:160])
    os.environ.pop("NCC_PIV_JIT", None)


if __name__ == "__main__":
    which = sys.argv[1:] or ["tm", "piv"]
    if "tm" in which:
        tm_surface()
    if "piv" in which:
        piv_surface()
