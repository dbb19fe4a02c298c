"""Top CUDA source lines of one kernel in an ncu report by warp-stall samples
(needs the source in the report: PF_JIT_DUMP=<dir> during the capture with
--import-source on).  usage: python tools/ncu_source_lines.py <rep> [n] [launch]"""
import csv
import os
import subprocess
import sys

rep = sys.argv[1]
n = int(sys.argv[2]) if len(sys.argv) > 2 else 30
sel = ["--launch-skip", sys.argv[3], "--launch-count", "1"] if len(sys.argv) > 3 else []
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"] + sel,
                     capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
lines, head, fname = [], None, "?"
for r in rows:
    if r and r[0] == "File Path":
        fname = os.path.basename(r[1])
        continue
    if r and r[0] == "Line No":
        head = r
        continue
    if head is None or not r or not r[0]:
        continue  # SASS rows (no CUDA line number)
    try:
        i = head.index("Warp Stall Sampling (All Samples)")
        samp = float(r[i] or 0)
    except (ValueError, IndexError):
        continue
    st = {}
    for j, c in enumerate(head):
        if c.startswith("stall_") and "Not Issued" not in c and j < len(r):
            try:
                st[c[6:]] = float(r[j] or 0)
            except ValueError:
                pass
    lines.append((samp, fname, r[0], r[1].strip(), st))
tot = sum(x[0] for x in lines) or 1.0
print(f"{os.path.basename(rep)}: {tot:.0f} stall samples over {len(lines)} source lines; top {n}")
for samp, f, ln, src, st in sorted(lines, key=lambda x: -x[0])[:n]:
    top = sorted(st.items(), key=lambda kv: -kv[1])[:2]
    print(f"{samp / tot:6.2%}  {f}:{ln:<5} {src[:80]:80s}  " + ", ".join(f"{k} {v / max(samp, 1):.0%}" for k, v in top))
