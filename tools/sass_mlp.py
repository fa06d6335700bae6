"""SASS memory-level-parallelism check: for every global load / returning atomic, how
many other global loads are issued between it and the first instruction that reads its
destination register (0 everywhere in a run = the loads are serialised).

    cuobjdump -sass lib.so | python tools/sass_mlp.py <kernel-substring>
"""
import re
import sys

name = sys.argv[1]
lines, on = [], False
for l in sys.stdin:
    if "Function :" in l:
        on = name in l
        continue
    m = re.match(r"\s*/\*([0-9a-f]{4,})\*/\s+(.*?);", l)
    if on and m:
        lines.append((m.group(1), m.group(2).strip()))
MEM = re.compile(r"\b(LDG|ATOMG|LD)\b[.\w]*\s+(?:PT,\s*)?(R\d+)")
out = []
for i, (addr, ins) in enumerate(lines):
    m = MEM.search(ins)
    if not m:
        continue
    rd = m.group(2)
    between = 0
    use = None
    for j in range(i + 1, min(len(lines), i + 400)):
        ins2 = lines[j][1]
        body = ins2.split(None, 1)[1] if " " in ins2 else ""
        srcs = body.split(",", 1)[1] if "," in body else body
        if re.search(r"\b" + rd + r"\b", srcs) or (MEM.search(ins2) and MEM.search(ins2).group(2) == rd):
            use = j
            break
        if MEM.search(ins2):
            between += 1
    out.append((addr, between, ins[:90]))
for addr, b, ins in out:
    print(f"{addr} in-flight-after={b:3d}  {ins}")
