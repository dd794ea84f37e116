#!/usr/bin/env python3
"""Summarise an ncu --metrics gpu__time_duration.sum launch list (CSV) per kernel."""
import collections, csv, sys

rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 10]
h = rows[0]
ik, iv, iu = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
tot = collections.defaultdict(float)
cnt = collections.Counter()
for r in rows[1:]:
    v = float(r[iv].replace(",", ""))
    v = v / 1e6 if r[iu] == "ns" else v / 1e3 if r[iu] in ("us", "usecond") else v
    tot[r[ik]] += v
    cnt[r[ik]] += 1
T = sum(tot.values())
print("| kernel | launches | total ms | mean ms | share |\n|---|---|---|---|---|")
for k, v in sorted(tot.items(), key=lambda kv: -kv[1]):
    print(f"| `{k}` | {cnt[k]} | {v:.3f} | {v / cnt[k]:.4f} | {v / T * 100:.1f}% |")
