import glob, json, os
os.chdir(os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", "gpurun_out"))
for f in sorted(glob.glob("sched_tests_*.log")):
    print(f, open(f).read().strip().splitlines()[-2:])
for f in sorted(glob.glob("sched_cfg*.json")):
    try:
        d = json.load(open(f)); r = d["roofline"]
        print(f, round(d["value"] / 1e9, 3), round(d["ms_per_step"], 4), round(r["kernel_ms"], 4), round(r["frac"], 3), d["correct"], d["clocks"]["sm_mhz"])
    except Exception as e:
        print(f, "ERR", e)
for f in sorted(glob.glob("tl*.json")):
    s = open(f).read(); s = s[s.index("{"):]
    d = json.loads(s); print(f, d["spans_us"])
    for k in d["best"]["kernels"]:
        print("   ", k["start_us"], k["end_us"], k["dur_us"], k["name"])
