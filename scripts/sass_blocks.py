#!/usr/bin/env python3
"""Split cuobjdump SASS of one function into basic blocks; print opcode mix per block."""
import collections, re, sys
lines = [l for l in open(sys.argv[1]) if re.match(r"\s*/\*[0-9a-f]{4,}\*/", l)]
ins = []
for l in lines:
    m = re.match(r"\s*/\*([0-9a-f]+)\*/\s*(.*?);", l)
    if m: ins.append((int(m.group(1), 16), m.group(2).strip()))
targets = {int(t, 16) for _, s in ins for t in re.findall(r"BRA[^0]*?(0x[0-9a-f]+)", s)}
blocks, cur = [], []
for a, s in ins:
    if a in targets and cur: blocks.append(cur); cur = []
    cur.append((a, s))
    if re.search(r"\bBRA\b|EXIT|BAR\.SYNC", s): blocks.append(cur); cur = []
if cur: blocks.append(cur)
minfp = int(sys.argv[2]) if len(sys.argv) > 2 else 8
for b in blocks:
    ops = collections.Counter((s.split()[1] if s.startswith("@") else s.split()[0]).split(".")[0] for _, s in b)
    fp = sum(v for k, v in ops.items() if k in ("FFMA2", "FMUL2", "FFMA", "FMUL", "FADD"))
    if fp >= minfp:
        print(f"{b[0][0]:#06x}-{b[-1][0]:#06x} n={len(b)} fp={fp} other={len(b)-fp}: " + ", ".join(f"{k}{v}" for k, v in ops.most_common() if k not in ("FFMA2","FMUL2")))
