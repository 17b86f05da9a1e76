#!/usr/bin/env python
"""Per-stage device times (plan NCC_F_TIMING events) of cfg2 (TM) and cfg3/cfg4 (PIV):
median over reps of prep / window sums / numerator / finalize / total.  Env knobs
(NCC_BOX_TWO_PASS, NCC_FORCE_SPLIT, ...) apply.  Usage: python tools/stage_times.py [cfg ...]"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_ipps_moorelk13_b200.api import MatchPlan, PivPlan  # noqa: E402

DEV = torch.device("cuda", 0)


def med(plan, fn, reps):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    rows = []
    for _ in range(reps):
        fn()
        t = plan.timing()
        rows.append((t.prep_ms, t.stats_ms, t.numerator_ms, t.finalize_ms, t.total_ms))
    return dict(zip(("prep_ms", "stats_ms", "numerator_ms", "finalize_ms", "total_ms"),
                    np.median(np.array(rows), axis=0).tolist()))


def main():
    cfgs = [int(c) for c in sys.argv[1:]] or [2, 3]
    env = {k: v for k, v in os.environ.items() if k.startswith("NCC_")}
    for cfg in cfgs:
        c = synth.CONFIGS[cfg]
        if c["kind"] == "tm":
            img, T, _, _ = synth.tm_inputs(cfg)
            d_img, d_t = torch.from_numpy(img).to(DEV), torch.from_numpy(T).to(DEV)
            with MatchPlan(c["H"], c["W"], c["h"], c["w"], timing=True) as plan:
                r = med(plan, lambda: plan.match(d_img, d_t), 20)
                name = plan.info.variant_name.decode()
        else:
            P = 1 if cfg == 3 else 16
            A = torch.rand((P, c["H"], c["W"]), device=DEV)
            B = torch.rand((P, c["H"], c["W"]), device=DEV)
            with PivPlan(c["H"], c["W"], c["h"], c["m"], c["step"], pairs=P, timing=True) as plan:
                r = med(plan, lambda: plan.correlate(A, B, scores=False), 10)
                name = plan.info.variant_name.decode()
        print(json.dumps(dict(cfg=cfg, variant=name, env=env, **r)), flush=True)


if __name__ == "__main__":
    main()
