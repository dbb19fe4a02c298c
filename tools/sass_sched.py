"""Static schedule of the loops of one kernel in a cubin: for every loop
(backward branch) the instruction count, the fp64 / LDS / LDG / BAR counts
and the sum of the compiler's stall counts (control bits of the SASS), i.e.
the cycles ONE warp needs per iteration if every variable-latency wait were
free.  Compared with the fp64 pipe time of the same iteration (2 cycles per
warp fp64 instruction on a 16-lane SM sub-partition) it says how many warps
per sub-partition the schedule needs to keep the fp64 pipe busy.
usage: python tools/sass_sched.py <cubin> <kernel name>"""
import re
import subprocess
import sys

cub, kname = sys.argv[1], sys.argv[2]
sass = subprocess.run(["cuobjdump", "-sass", cub], capture_output=True, text=True).stdout
funcs = re.split(r"\n\s+Function : ", sass)
body = None
for f in funcs[1:]:
    if f.split("\n", 1)[0].strip() == kname:
        body = f
assert body, kname
lines = body.splitlines()
ins = []
i = 0
while i < len(lines):
    m = re.match(r"\s+/\*([0-9a-f]{4,})\*/\s+(.*?);\s+/\* (0x[0-9a-f]+) \*/", lines[i])
    if m:
        hi = int(re.search(r"/\* (0x[0-9a-f]+) \*/", lines[i + 1]).group(1), 16)
        txt = m.group(2).strip()
        op = re.sub(r"^@!?U?P\w+\s+", "", txt).split()[0]
        ins.append(dict(addr=int(m.group(1), 16), txt=txt, op=op, stall=(hi >> 41) & 0xF,
                        yld=(hi >> 45) & 1, wait=(hi >> 52) & 0x3F))
        i += 2
    else:
        i += 1
by_addr = {x["addr"]: k for k, x in enumerate(ins)}
loops = []
for k, x in enumerate(ins):
    if x["op"].startswith("BRA"):
        m = re.search(r"0x([0-9a-f]+)", x["txt"])
        if m and int(m.group(1), 16) < x["addr"]:
            loops.append((by_addr[int(m.group(1), 16)], k))
fp64 = ("DFMA", "DADD", "DMUL")
for a, b in loops:
    seg = ins[a:b + 1]
    cnt = lambda p: sum(1 for x in seg if x["op"].split(".")[0] in p)
    st = sum(x["stall"] for x in seg)
    nf = cnt(fp64)
    print(f"loop {ins[a]['addr']:#06x}-{ins[b]['addr']:#06x}: {len(seg)} instr, fp64 {nf}, MUFU {cnt(('MUFU',))}, "
          f"LDS {cnt(('LDS',))}, STS {cnt(('STS',))}, LDL {cnt(('LDL',))}, STL {cnt(('STL',))}, LDG {cnt(('LDG',))}, STG {cnt(('STG',))}, BAR {cnt(('BAR',))}, "
          f"stall sum {st} cyc, fp64 pipe {2 * nf} cyc, waits on scoreboards {sum(1 for x in seg if x['wait'])}")
