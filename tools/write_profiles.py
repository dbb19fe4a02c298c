"""Copy the evidence of one GPU session into profiles/ (tracked):
bench line, ncu launch list, ncu --set full summaries of the sweeps (key
metrics, stall reasons, dynamic instruction mix), fp64 micro-benchmarks, and
profiles/ncu_summary.json (dram bytes per launch, read by bench.py).
usage: python tools/write_profiles.py gpurun_out/<dir> <round-tag>"""
import collections
import csv
import json
import os
import re
import shutil
import subprocess
import sys

src, tag = sys.argv[1], sys.argv[2]
dst = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "profiles")
os.makedirs(dst, exist_ok=True)
for name, out in (("bench.json", f"{tag}_bench.json"), ("bench_strong.json", f"{tag}_bench_strong.json"), ("launches.csv", f"{tag}_launches.csv"),
                  ("fp64_micro.json", f"{tag}_fp64_micro.json"), ("pytest_gpu.log", f"{tag}_pytest_gpu.log"),
                  ("smoke.log", f"{tag}_smoke.log"), ("nvidia-smi.txt", f"{tag}_nvidia-smi.txt")):
    p = os.path.join(src, name)
    if os.path.exists(p):
        shutil.copy(p, os.path.join(dst, out))

KEYS = ["gpu__time_duration.sum", "launch__registers_per_thread", "launch__occupancy_limit_registers",
        "launch__occupancy_limit_shared_mem", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "l1tex__throughput.avg.pct_of_peak_sustained_active",
        "dram__bytes_read.sum", "dram__bytes_write.sum", "dram__throughput.avg.pct_of_peak_sustained_elapsed",
        "lts__t_sector_hit_rate.pct", "smsp__inst_executed.sum", "smsp__sass_inst_executed_op_global_ld.sum",
        "smsp__sass_inst_executed_op_shared_ld.sum", "smsp__sass_inst_executed_op_local_ld.sum"]
summary = {}
# (report, launch in it, name): prof_p2jit holds the specialised P2 phi- and
# mu-sweep (both named pf_p2_jit), launches 0 and 1
JOBS = [("mu", 0, "mu"), ("phi", 0, "phi"), ("ghost", 0, "ghost"), ("p2phi", 0, "p2phi"), ("p2mu", 0, "p2mu"),
        ("p2jit", 0, "p2jitphi"), ("p2jit", 1, "p2jitmu")]
for rname, li, kern in JOBS:
    rep = os.path.join(src, f"prof_{rname}.ncu-rep")
    if not os.path.exists(rep):
        continue
    sel = ["--launch-skip", str(li), "--launch-count", "1"]
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"] + sel, capture_output=True, text=True).stdout
    rows = list(csv.reader(raw.splitlines()))
    h, u, v = rows[0], rows[1], rows[2]
    m = {n: (v[i], u[i]) for i, n in enumerate(h)}
    lines = [f"ncu --set full summary: {m.get('Kernel Name', ('?',))[0]}  (session {os.path.basename(src)})", ""]
    for k in KEYS:
        if k in m:
            lines.append(f"  {k:70s} {m[k][0]} {m[k][1]}")
    # hardware-counted fp64 work (S§8(d) D.5): DADD + DMUL + 2 DFMA thread
    # instructions, per interior cell of the launch (256^3 bench block)
    hw = {}
    try:
        cyc = float(m["smsp__cycles_elapsed.avg"][0])
        tsec = float(m["gpu__time_duration.sum"][0]) * {"us": 1e-6, "ms": 1e-3, "ns": 1e-9}[m["gpu__time_duration.sum"][1]]
        cells = 256 ** 3
        for op in ("dadd", "dmul", "dfma"):
            hw[op] = float(m[f"smsp__sass_thread_inst_executed_op_{op}_pred_on.sum.per_cycle_elapsed"][0]) * cyc / cells
        hw["flop_per_cell"] = hw["dadd"] + hw["dmul"] + 2 * hw["dfma"]
        hw["tflops"] = hw["flop_per_cell"] * cells / tsec / 1e12
        lines += ["", f"  hardware-counted fp64 per cell (256^3 launch): DADD {hw['dadd']:.1f}, DMUL {hw['dmul']:.1f}, "
                      f"DFMA {hw['dfma']:.1f} -> {hw['flop_per_cell']:.1f} flop/cell, {hw['tflops']:.2f} TFLOP/s "
                      f"(rsqrt / rcp seeds on MUFU not counted)"]
    except (KeyError, ValueError):
        pass
    st = {n.replace("smsp__average_warps_issue_stalled_", "").replace("_per_issue_active.ratio", ""): float(v[i] or 0)
          for i, n in enumerate(h)
          if n.startswith("smsp__average_warps_issue_stalled") and n.endswith("per_issue_active.ratio")}
    lines += ["", "  warp stall reasons (cycles per issued instruction):"]
    lines += [f"    {k:28s} {x:6.2f}" for k, x in sorted(st.items(), key=lambda kv: -kv[1]) if x > 0.05]
    srcp = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"] + sel,
                          capture_output=True, text=True).stdout
    srows = list(csv.reader(srcp.splitlines()))
    if len(srows) > 2:
        hh = srows[1]
        iE = hh.index("Instructions Executed")
        ops = collections.Counter()
        for r in srows[2:]:
            mm = re.match(r"(@!?U?P\w+\s+)?([A-Z0-9_]+)", r[1].strip())
            if mm:
                ops[mm.group(2)] += int(r[iE] or 0)
        tot = sum(ops.values())
        fp64 = sum(ops[o] for o in ("DFMA", "DMUL", "DADD", "DSETP", "DMNMX", "MUFU"))
        lines += ["", f"  dynamic instruction mix (warp-level, total {tot}, fp64-pipe share {fp64 / max(tot, 1):.1%}):"]
        lines += [f"    {k:10s} {c / tot:6.1%}" for k, c in ops.most_common(20)]
        # stall samples per code region (regions end at a CTA barrier)
        iS = hh.index("Warp Stall Sampling (All Samples)")
        scol = [c for c in hh if c.startswith("stall_") and "Not Issued" not in c]
        regs, cur = [], {"n": 0, "samples": 0.0, "exec": 0.0, "st": collections.Counter()}
        for r in srows[2:]:
            cur["n"] += 1
            cur["samples"] += float(r[iS] or 0)
            cur["exec"] += float(r[iE] or 0)
            for c in scol:
                cur["st"][c[6:]] += float(r[hh.index(c)] or 0)
            if "BAR.SYNC" in r[1] or re.search(r"\bEXIT\b", r[1]):
                cur["end"] = r[1].strip()[:28]
                regs.append(cur)
                cur = {"n": 0, "samples": 0.0, "exec": 0.0, "st": collections.Counter()}
        ts = sum(x["samples"] for x in regs) or 1.0
        te = sum(x["exec"] for x in regs) or 1.0
        lines += ["", "  stall samples by code region (region = SASS up to a BAR.SYNC / EXIT):"]
        for x in regs:
            if x["samples"] / ts < 0.02:
                continue
            top = ", ".join(f"{k} {v / x['samples']:.0%}" for k, v in x["st"].most_common(4))
            lines.append(f"    {x['n']:4d} instr ending '{x['end']}': {x['samples'] / ts:5.1%} of samples, "
                         f"{x['exec'] / te:5.1%} of executed; top: {top}")
    open(os.path.join(dst, f"{tag}_ncu_{kern}.txt"), "w").write("\n".join(lines) + "\n")
    rd = float(m["dram__bytes_read.sum"][0]) * {"Gbyte": 1e9, "Mbyte": 1e6, "Kbyte": 1e3, "byte": 1}[m["dram__bytes_read.sum"][1]]
    wr = float(m["dram__bytes_write.sum"][0]) * {"Gbyte": 1e9, "Mbyte": 1e6, "Kbyte": 1e3, "byte": 1}[m["dram__bytes_write.sum"][1]]
    summary[f"{kern}_sweep"] = {"dram_bytes_per_launch": rd + wr, "dram_read": rd, "dram_write": wr,
                                "session": os.path.basename(src), "round": tag}
    if hw:
        summary[f"{kern}_sweep"].update({"hw_flop_per_cell": hw["flop_per_cell"], "hw_tflops": hw["tflops"]})
if summary:
    p = os.path.join(dst, "ncu_summary.json")
    old = json.load(open(p)) if os.path.exists(p) else {}
    old.update(summary)
    json.dump(old, open(p, "w"), indent=1)
print("wrote", sorted(os.listdir(dst)))
