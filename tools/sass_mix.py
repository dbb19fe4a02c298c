"""Opcode histogram of one kernel in libpf.so (static SASS count).
usage: python tools/sass_mix.py <substring of mangled name> [lib]"""
import collections
import re
import subprocess
import sys

pat = sys.argv[1]
lib = sys.argv[2] if len(sys.argv) > 2 else "paper_conf_sc_0003hehshhkwnr19_b200/libpf.so"
sass = subprocess.run(["cuobjdump", "-sass", lib], capture_output=True, text=True).stdout
funcs = re.split(r"\n\s+Function : ", sass)
for f in funcs[1:]:
    name = f.split("\n", 1)[0].strip()
    if pat not in name:
        continue
    ops = collections.Counter()
    n = 0
    for l in f.splitlines():
        m = re.match(r"\s+/\*[0-9a-f]{4,}\*/\s+(@!?U?P\w+\s+)?([A-Z0-9_.]+)", l)
        if m:
            ops[m.group(2).split(".")[0]] += 1
            n += 1
    print(name, "total", n)
    print("  ".join(f"{k}:{v}" for k, v in ops.most_common(45)))
    break
