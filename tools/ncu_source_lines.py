"""Top CUDA source lines of one kernel in an ncu report by warp-stall samples
(needs the source in the report: PF_JIT_DUMP=<dir> during the capture with
--import-source on).  usage: python tools/ncu_source_lines.py <rep> [n] [launch]"""
import csv
import subprocess
import sys

rep = sys.argv[1]
n = int(sys.argv[2]) if len(sys.argv) > 2 else 30
sel = ["--launch-skip", sys.argv[3], "--launch-count", "1"] if len(sys.argv) > 3 else []
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda"] + sel,
                     capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
hi = [i for i, r in enumerate(rows) if "Source" in r and any("Warp Stall Sampling" in c for c in r)]
if not hi:
    sys.exit("no source page (was the source imported?)")
h = rows[hi[0]]
data = rows[hi[0] + 1:]
iS = h.index("Warp Stall Sampling (All Samples)")
iL = h.index("# Line") if "# Line" in h else 0
iSrc = h.index("Source")
scol = [c for c in h if c.startswith("stall_") and "Not Issued" not in c]
tot = sum(float(r[iS] or 0) for r in data if len(r) > iS)
best = sorted((r for r in data if len(r) > iS and float(r[iS] or 0) > 0), key=lambda r: -float(r[iS]))[:n]
print(f"{rep}: {tot:.0f} stall samples; top {n} source lines")
for r in best:
    st = sorted(((c[6:], float(r[h.index(c)] or 0)) for c in scol), key=lambda x: -x[1])[:2]
    print(f"{float(r[iS]) / tot:6.2%}  line {r[iL]:>5}  {r[iSrc].strip()[:90]:90s}  {', '.join(f'{k} {v / float(r[iS]):.0%}' for k, v in st)}")
