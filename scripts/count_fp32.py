#!/usr/bin/env python3
"""n_fp32 of SURVEY §8(d) measured from an ncu report of ONE HHC row launch:
FP32-pipe lane operations (predicated-on thread instructions of FFMA/FMUL/FADD,
x2 for the packed FFMA2/FMUL2/FADD2; MUFU and FCHK excluded) divided by the
interior updates that launch performs.

    count_fp32.py REPORT.ncu-rep UPDATES_PER_LAUNCH
"""
import collections
import csv
import io
import subprocess
import sys

rep, upd = sys.argv[1], float(sys.argv[2])
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr = rows[1]
ia, ip = hdr.index("Source"), hdr.index("Predicated-On Thread Instructions Executed")
ops = collections.Counter()
for r in rows[2:]:
    if len(r) <= ip:
        continue
    s = r[ia].strip()
    op = (s.split()[1] if s.startswith("@") else s.split()[0]) if s else ""
    try:
        ops[op.split(".")[0]] += int(r[ip])
    except ValueError:
        pass
single = ("FFMA", "FMUL", "FADD")
packed = ("FFMA2", "FMUL2", "FADD2")
lane = sum(ops[o] for o in single) + 2 * sum(ops[o] for o in packed)
print(f"report {rep}")
for o in single + packed + ("MUFU", "FCHK", "FSETP"):
    print(f"  {o:6s} {ops[o]:16d} thread instr ({ops[o] / upd:7.3f} per update)")
print(f"FP32-pipe lane ops {lane} / {upd:.6g} updates = n_fp32 {lane / upd:.2f}")
