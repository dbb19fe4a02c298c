"""Print bench lines and key ncu metrics of a gpurun_out/<tag> directory."""
import csv
import glob
import json
import os
import subprocess
import sys

d = sys.argv[1]
for f in sorted(glob.glob(os.path.join(d, "bench*.json"))):
    try:
        r = json.loads(open(f).read().strip().splitlines()[-1])
        k = {a: (round(b, 4) if isinstance(b, float) else b) for a, b in r.get("kernels", {}).items()}
        print(os.path.basename(f), round(r["value"]), "MLUP/s", round(r["ms_per_step"], 4), "ms/step",
              "frac_R", round(r["step_roofline"]["frac"], 4), "mu_frac", round(r["roofline"]["frac"] or 0, 4), k)
    except Exception as e:
        print(f, "ERR", e)
p = os.path.join(d, "pytest_gpu.log")
if os.path.exists(p):
    print([l for l in open(p).read().splitlines() if "passed" in l or "failed" in l or "exit" in l][-2:])
want = ["gpu__time_duration.sum", "launch__registers_per_thread",
        "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active",
        "l1tex__throughput.avg.pct_of_peak_sustained_active", "smsp__inst_executed.sum",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "dram__bytes_read.sum", "dram__bytes_write.sum"]
for rep in sorted(glob.glob(os.path.join(d, "*.ncu-rep"))):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    if len(rows) < 3:
        continue
    h, units, v = rows[0], rows[1], rows[2]
    print("==", os.path.basename(rep))
    print("  ", {n: (v[i] + " " + units[i]) for i, n in enumerate(h) if n in want})
    st = {n.replace("smsp__average_warps_issue_stalled_", "").replace("_per_issue_active.ratio", ""): float(v[i] or 0)
          for i, n in enumerate(h) if n.startswith("smsp__average_warps_issue_stalled") and n.endswith("per_issue_active.ratio")}
    print("   stalls", {k: round(x, 2) for k, x in sorted(st.items(), key=lambda kv: -kv[1])[:7]})
lp = os.path.join(d, "launches.csv")
if os.path.exists(lp):
    import collections
    lines = open(lp).read().splitlines()
    st = [i for i, l in enumerate(lines) if l.startswith('"ID"')]
    if st:
        agg = collections.defaultdict(list)
        for r in csv.DictReader(lines[st[0]:]):
            agg[r["Kernel Name"][:60]].append(float(r["Metric Value"]))
        tot = sum(sum(v) for v in agg.values())
        print("== launch list (ncu, serialized)")
        for k, v in sorted(agg.items(), key=lambda kv: -sum(kv[1])):
            print(f"   {sum(v)/1e3:9.1f} us  {100*sum(v)/tot:5.1f}%  n={len(v):3d} avg={sum(v)/len(v)/1e3:8.1f} us  {k}")
