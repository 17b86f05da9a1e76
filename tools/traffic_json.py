#!/usr/bin/env python
"""Write profiles/roofline_traffic.json (bench.py's roofline.traffic) from the round's ncu --set
full summaries: dram__bytes_read.sum + dram__bytes_write.sum per launch of the dominant kernel.
Usage: python tools/traffic_json.py <round> <dir with prof_cfg2.json prof_cfg5.json prof_piv3.json prof_piv4.json>"""
import json
import os
import sys

UNIT = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}


def nbytes(rec, key):
    v = rec[key]
    return float(v["value"]) * UNIT[v["unit"]]


def main():
    rnd, d = sys.argv[1], sys.argv[2]
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    path = os.path.join(root, "profiles", "roofline_traffic.json")
    out = json.load(open(path)) if os.path.exists(path) else {}
    src = dict(out.get("source", {}))
    out["note"] = (f"dram__bytes_read.sum + dram__bytes_write.sum per launch of the dominant (numerator) kernel, "
                   f"from one ncu --set full capture (profiles/{rnd}_ncu_full_*.json; *_tc = tm_tc_kernel). "
                   f"cfg4 is per pair (capture: 8-pair launch); bench.py multiplies by the pairs of its launches; "
                   f"'source' names the round each figure was captured in")
    for key, name, per in (("cfg2_tc", "prof_cfg2.json", 1), ("cfg5_tc", "prof_cfg5.json", 1),
                           ("cfg3", "prof_piv3.json", 1), ("cfg4_tc_per_pair", "prof_piv4.json", 8),
                           ("cfg4_per_pair", "prof_piv4cc.json", 8)):
        p = os.path.join(d, name)
        if not os.path.exists(p):
            continue
        rec = json.load(open(p))[0]
        out[key] = (nbytes(rec, "dram__bytes_read.sum") + nbytes(rec, "dram__bytes_write.sum")) / per
        src[key] = rnd
    for key in out:
        if key not in ("note", "source") and key not in src:
            src[key] = "r01"
    out["source"] = src
    json.dump(out, open(path, "w"), indent=1)
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
