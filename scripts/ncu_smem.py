#!/usr/bin/env python3
"""Shared-memory wavefronts per SASS instruction from an ncu report's source page:
the instructions with the most excess (conflict) wavefronts and the totals."""
import csv, io, subprocess, sys

rep = sys.argv[1]
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
h = rows[1]
ix = {k: h.index(k) for k in ("Source", "L1 Wavefronts Shared", "L1 Wavefronts Shared Ideal",
                              "L1 Wavefronts Shared Excessive", "Instructions Executed")}
recs = []
for r in rows[2:]:
    if len(r) < len(h):
        continue
    try:
        wf, ideal, exc = (float(r[ix[k]] or 0) for k in ("L1 Wavefronts Shared", "L1 Wavefronts Shared Ideal",
                                                        "L1 Wavefronts Shared Excessive"))
    except ValueError:
        continue
    if wf > 0:
        recs.append((exc, wf, ideal, r[ix["Source"]].strip(), r[ix["Instructions Executed"]]))
tw = sum(x[1] for x in recs); ti = sum(x[2] for x in recs); te = sum(x[0] for x in recs)
print(f"shared wavefronts {tw:.3e}, ideal {ti:.3e}, excessive {te:.3e} ({te / max(tw, 1):.1%})")
by_op = {}
for exc, wf, ideal, src, n in recs:
    op = src.split()[0] if src else "?"
    a = by_op.setdefault(op, [0, 0, 0])
    a[0] += wf; a[1] += ideal; a[2] += exc
for op, (wf, ideal, exc) in sorted(by_op.items(), key=lambda kv: -kv[1][0])[:12]:
    print(f"  {op:14s} wavefronts {wf:.3e} ({wf / tw:.1%})  excessive {exc:.3e}")
for exc, wf, ideal, src, n in sorted(recs, reverse=True)[:12]:
    print(f"  excess {exc:.3e} of {wf:.3e}  {src[:70]}  (executed {n})")
