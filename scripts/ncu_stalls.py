#!/usr/bin/env python3
"""Per-source-line warp stall samples (top lines, with their main stall reasons) from an ncu report."""
import collections, csv, io, subprocess, sys
rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 30
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
f = hdr = cur = None
tot = collections.defaultdict(collections.Counter)
seen = set()
for r in csv.reader(io.StringIO(out)):
    if len(r) == 2 and r[0] == "File Path": f = r[1].split("/")[-1]; continue
    if len(r) <= 2: continue
    if r[0] == "Line No": hdr = r; continue
    if not hdr: continue
    if r[0] != "":
        try: cur = (f, int(r[0]), r[1].strip()[:64])
        except ValueError: pass
        continue
    if r[2] in seen: continue
    seen.add(r[2])
    d = dict(zip(hdr, r))
    for k, v in d.items():
        if (k.startswith("stall_") and "Not Issued" not in k) or k == "Warp Stall Sampling (All Samples)":
            try: tot[cur][k] += int(v or 0)
            except ValueError: pass
T = sum(c["Warp Stall Sampling (All Samples)"] for c in tot.values()) or 1
print("total samples", T)
for key, c in sorted(tot.items(), key=lambda kv: -kv[1]["Warp Stall Sampling (All Samples)"])[:top]:
    n = c["Warp Stall Sampling (All Samples)"]
    st = sorted(((k[6:], v) for k, v in c.items() if k.startswith("stall_")), key=lambda kv: -kv[1])[:3]
    print(f"{n / T * 100:5.1f}% {key[0]}:{key[1]:4d} {key[2]:64s} " + " ".join(f"{k}={v / max(n,1) * 100:.0f}%" for k, v in st if v))
