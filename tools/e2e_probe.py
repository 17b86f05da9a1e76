"""Where the end-to-end (host buffers) time of one TM / PIV call goes:
python tools/e2e_probe.py tm CFG | piv CFG.

Times, with CUDA events on one stream (median of 20 after 5 warm-ups, no L2 flush): the pinned
host->device copy of the call's inputs alone (torch), the device-resident call, the host-buffer
call (ncc_match_host / piv_correlate_host) and the copy followed by the device call."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
import synth  # noqa: E402
from paper_conf_ipps_moorelk13_b200.api import MatchPlan, PivPlan  # noqa: E402

kind, cfg = sys.argv[1], int(sys.argv[2])
dev = torch.device("cuda", 0)
stream = torch.cuda.Stream(dev)


def timed(fn, n=20, w=5):
    for _ in range(w):
        fn()
    torch.cuda.synchronize()
    ts = []
    for _ in range(n):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        fn()
        e1.record(stream)
        e1.synchronize()
        ts.append(e0.elapsed_time(e1))
    ts.sort()
    return ts[len(ts) // 2]


out = {"kind": kind, "cfg": cfg, "graphs": os.environ.get("NCC_NO_GRAPH") is None}
c = synth.CONFIGS[cfg]
with torch.cuda.stream(stream):
    if kind == "tm":
        img, T, _, _ = synth.tm_inputs(cfg)
        d_img, d_t = torch.from_numpy(img).to(dev), torch.from_numpy(T).to(dev)
        h_img, h_t = torch.from_numpy(img).pin_memory(), torch.from_numpy(T).pin_memory()
        h_pk = torch.empty((1, 4), dtype=torch.int32).pin_memory()
        peaks = torch.empty((1, 4), dtype=torch.int32, device=dev)
        with MatchPlan(c["H"], c["W"], c["h"], c["w"]) as plan:
            out["variant"] = plan.info.variant_name.decode()
            out["h2d_ms"] = timed(lambda: (d_img.copy_(h_img, non_blocking=True), d_t.copy_(h_t, non_blocking=True)))
            out["h2d_img_ms"] = timed(lambda: d_img.copy_(h_img, non_blocking=True))
            out["h2d_tmpl_ms"] = timed(lambda: d_t.copy_(h_t, non_blocking=True))
            h_fresh = torch.empty(img.shape, dtype=torch.float32).pin_memory()
            h_fresh.copy_(torch.from_numpy(img))
            out["h2d_img_fresh_ms"] = timed(lambda: d_img.copy_(h_fresh, non_blocking=True))
            out["h_img_pinned"] = bool(h_img.is_pinned())
            out["device_ms"] = timed(lambda: plan.match(d_img, d_t, stream=stream, peaks=peaks))
            out["host_call_ms"] = timed(lambda: plan.match_host(h_img, h_t, h_pk, stream=stream))

            def copy_then_device():
                d_img.copy_(h_img, non_blocking=True)
                d_t.copy_(h_t, non_blocking=True)
                plan.match(d_img, d_t, stream=stream, peaks=peaks)
                h_pk.copy_(peaks, non_blocking=True)
            out["copy_then_device_ms"] = timed(copy_then_device)
            out["h2d_bytes"] = img.nbytes + T.nbytes
    else:
        P = 1 if cfg == 3 else int(sys.argv[3]) if len(sys.argv) > 3 else 16
        wl = dict(cfg=cfg, H=c["H"], W=c["W"], h=c["h"], w=c["w"], m=c["m"], step=c["step"], pairs=P, rank=0)
        A, B, _ = bench.piv_frames_device(wl, dev, torch)
        hA = torch.empty(A.shape, dtype=A.dtype).pin_memory()
        hA.copy_(A)
        hB = torch.empty(B.shape, dtype=B.dtype).pin_memory()
        hB.copy_(B)
        with PivPlan(c["H"], c["W"], c["h"], c["m"], c["step"], pairs=P, timing=True) as plan:
            out["variant"] = plan.info.variant_name.decode()
            Ky, Kx = plan.grid
            vec = torch.empty((P, Ky, Kx, 6), dtype=torch.int32, device=dev)
            hv = torch.empty(vec.shape, dtype=torch.int32).pin_memory()
            out["h2d_ms"] = timed(lambda: (A.copy_(hA, non_blocking=True), B.copy_(hB, non_blocking=True)))
            out["device_ms"] = timed(lambda: plan.correlate(A, B, stream=stream, vectors=vec))
            out["numerator_ms"] = plan.timing().numerator_ms
            out["host_call_ms"] = timed(lambda: plan.correlate_host(hA, hB, hv, stream=stream))
            out["h2d_bytes"] = 2 * A.numel() * 4
print(json.dumps(out))
