#!/usr/bin/env python3
"""Per-source-line executed warp instructions (all opcodes) from an ncu report."""
import collections, csv, io, subprocess, sys
rep = sys.argv[1]
thr = float(sys.argv[2]) if len(sys.argv) > 2 else 0.002
src = list(csv.reader(io.StringIO(subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source",
                                                  "cuda,sass"], capture_output=True, text=True).stdout)))
f = hdr = cur = None
per = collections.Counter()
seen = set()
for r in src:
    if len(r) == 2 and r[0] == "File Path":
        f = r[1].split("/")[-1]; continue
    if len(r) <= 2: continue
    if r[0] == "Line No": hdr = r; continue
    if not hdr: continue
    if r[0] != "":
        try: cur = (f, int(r[0]), r[1].strip()[:70])
        except ValueError: pass
        continue
    if r[2] in seen: continue
    seen.add(r[2])
    d = dict(zip(hdr, r))
    try: per[cur] += int(d["Instructions Executed"])
    except (ValueError, KeyError): pass
T = sum(per.values())
print("total", T)
for k, v in sorted(per.items(), key=lambda kv: (kv[0][0], kv[0][1])):
    if v / T > thr: print(f"{k[0]}:{k[1]:4d} {v / T * 100:5.1f}%  {k[2]}")
