#!/usr/bin/env python
"""Run one PIV config on the tensor-core kernel with NCC_PIV_TC_PROF and print the per-role wait
accounting (globaltimer ns summed over the CTAs, as fractions of each role's span).
  python tools/piv_tc_prof.py <cfg> <pairs>"""
import json
import os
import subprocess
import sys
import tempfile

import numpy as np

ROLES = {0: ("producers", ["img_full", "a_free"]), 8: ("prep", ["win_done(B slot)", "epi_done(stats)"]),
         16: ("epilogue", ["win_done", "drain", "st_full"]), 24: ("mma", ["a_full", "b_full", "d_free", "chunk_issue"])}


def main():
    cfg, P = sys.argv[1], sys.argv[2]
    path = os.path.join(tempfile.mkdtemp(), "ptc.bin")
    env = dict(os.environ, NCC_PIV_TC_PROF=path)
    here = os.path.dirname(os.path.abspath(__file__))
    subprocess.run([sys.executable, os.path.join(here, "piv_one.py"), cfg, P], env=env, check=True)
    raw = np.fromfile(path, dtype=np.uint64)
    ntr = 3 * 2048
    a = raw[:-ntr].reshape(-1, 32).astype(np.float64)
    tr = raw[-ntr:].reshape(-1, 3).astype(np.float64)
    tr = tr[tr[:, 0] > 0]
    act = a[a[:, 0] > 0]
    out = {"cfg": int(cfg), "pairs": int(P), "ctas": int(len(act))}
    for base, (name, keys) in ROLES.items():
        tot = act[:, base].sum()
        out[name] = {"span_ms_mean": round(act[:, base].mean() / 1e6, 4)}
        for k, key in enumerate(keys):
            out[name][key] = round(act[:, base + 1 + k].sum() / tot, 4) if tot else None
    if len(tr) > 10:  # CTA 0's first chunks (last call): wait, issue, and chunk-to-chunk times (cycles)
        t0 = tr[:, 0] - tr[0, 0]
        out["trace"] = {"wait_med": float(np.median(tr[:, 1] - tr[:, 0])), "issue_med": float(np.median(tr[:, 2] - tr[:, 1])),
                        "period_med": float(np.median(np.diff(tr[:, 0]))),
                        "first": [[int(x) for x in (t0[i], tr[i, 1] - tr[i, 0], tr[i, 2] - tr[i, 1])] for i in range(0, 40)]}
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
