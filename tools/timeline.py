#!/usr/bin/env python
"""GPU timeline of one execute call (kernel start/end per stream, CUPTI via torch.profiler):
where the step's time goes when several streams overlap.  L2 is flushed before every call, as
in bench.py.  Usage: python tools/timeline.py [cfg] [reps]   (cfg 2/5 TM, 3/4 PIV; env knobs apply)"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402
from torch.profiler import ProfilerActivity, profile  # noqa: E402

import synth  # noqa: E402
from paper_conf_ipps_moorelk13_b200.api import MatchPlan, PivPlan  # noqa: E402

DEV = torch.device("cuda", 0)


def main():
    cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 2
    reps = int(sys.argv[2]) if len(sys.argv) > 2 else 5
    c = synth.CONFIGS[cfg]
    flush = torch.empty(512 * 1024 * 1024 // 4, dtype=torch.float32, device=DEV)
    if c["kind"] == "tm":
        img, T, _, _ = synth.tm_inputs(cfg)
        d_img, d_t = torch.from_numpy(img).to(DEV), torch.from_numpy(T).to(DEV)
        plan = MatchPlan(c["H"], c["W"], c["h"], c["w"])
        call = lambda: plan.match(d_img, d_t)  # noqa: E731
        if os.environ.get("TL_HOST"):  # the host-buffer entry point (copies in the timeline)
            h_img, h_t = torch.from_numpy(img).pin_memory(), torch.from_numpy(T).pin_memory()
            h_pk = torch.empty((1, 4), dtype=torch.int32).pin_memory()
            call = lambda: plan.match_host(h_img, h_t, h_pk)  # noqa: E731
    else:
        P = 1 if cfg == 3 else 8
        A = torch.rand((P, c["H"], c["W"]), device=DEV)
        B = torch.rand((P, c["H"], c["W"]), device=DEV)
        plan = PivPlan(c["H"], c["W"], c["h"], c["m"], c["step"], pairs=P)
        call = lambda: plan.correlate(A, B, scores=False)  # noqa: E731
    for _ in range(3):
        flush.fill_(1.0)
        call()
    torch.cuda.synchronize()
    with profile(activities=[ProfilerActivity.CUDA, ProfilerActivity.CPU]) as prof:
        for _ in range(reps):
            flush.fill_(1.0)
            call()
        torch.cuda.synchronize()
    evs = [e for e in prof.events() if e.device_type.name == "CUDA" or "Memcpy" in e.name]
    evs.sort(key=lambda e: e.time_range.start)
    # split into steps at each flush kernel
    steps, cur = [], None
    for e in evs:
        if "FillFunctor" in e.name:
            if cur:
                steps.append(cur)
            cur = {"flush_end": e.time_range.end, "k": []}
        elif cur is not None:
            cur["k"].append(e)
    if cur:
        steps.append(cur)
    out = []
    for st in steps:
        t0 = st["flush_end"]
        ks = [{"name": e.name.split("(")[0][-48:], "stream": getattr(e, "device_index", 0),
               "start_us": round(e.time_range.start - t0, 2), "end_us": round(e.time_range.end - t0, 2),
               "dur_us": round(e.time_range.end - e.time_range.start, 2)} for e in st["k"]]
        out.append({"span_us": round(max(k["end_us"] for k in ks), 2), "kernels": ks})
    best = min(out, key=lambda s: s["span_us"])
    print(json.dumps({"cfg": cfg, "variant": plan.info.variant_name.decode(),
                      "spans_us": [s["span_us"] for s in out], "best": best}, indent=1))
    plan.close()


if __name__ == "__main__":
    main()
