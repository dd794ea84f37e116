#!/usr/bin/env python3
"""Summarise an ncu report: key SOL/scheduler metrics, stall reasons, opcode mix
and the source lines with the most non-FP instructions (per block-level if
--units is given)."""
import collections, csv, io, subprocess, sys

rep = sys.argv[1]
units = float(sys.argv[2]) if len(sys.argv) > 2 else 1.0


def ncu(*args):
    return subprocess.run(["ncu", "-i", rep, *args], capture_output=True, text=True).stdout


rows = list(csv.reader(io.StringIO(ncu("--page", "details", "--csv"))))
h = rows[0]
want = ["Duration", "Elapsed Cycles", "Executed Ipc Active", "Issue Slots Busy", "No Eligible",
        "Eligible Warps Per Scheduler", "Warp Cycles Per Issued Instruction", "Executed Instructions",
        "L1/TEX Cache Throughput", "DRAM Throughput", "Registers Per Thread", "Achieved Active Warps Per SM",
        "Compute (SM) Throughput", "Memory Throughput"]
for r in rows[1:]:
    d = dict(zip(h, r))
    if d.get("Metric Name") in want:
        print(f"{d['Metric Name']:40s} {d['Metric Value']:>16s} {d['Metric Unit']}")
raw = list(csv.reader(io.StringIO(ncu("--page", "raw", "--csv"))))
d = dict(zip(raw[0], raw[2]))
st = sorted(((k.replace("smsp__pcsamp_warps_issue_stalled_", ""), float(v.replace(",", "") or 0))
             for k, v in d.items() if k.startswith("smsp__pcsamp_warps_issue_stalled") and not k.endswith("not_issued")),
            key=lambda kv: -kv[1])
tot = sum(v for _, v in st) or 1
print("stalls:", ", ".join(f"{k} {v / tot * 100:.1f}%" for k, v in st[:9]))
for k in ["l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
          "smsp__inst_executed.sum"]:
    print(k, d.get(k), raw[1][raw[0].index(k)] if k in raw[0] else "")
src = list(csv.reader(io.StringIO(ncu("--page", "source", "--csv", "--print-source", "cuda,sass"))))
f = hdr = cur = None
per = collections.defaultdict(collections.Counter)
ops = collections.Counter()
seen = set()
for r in src:
    if len(r) == 2 and r[0] == "File Path":
        f = r[1].split("/")[-1]
        continue
    if len(r) <= 2:
        continue
    if r[0] == "Line No":
        hdr = r
        continue
    if not hdr:
        continue
    if r[0] != "":
        try:
            cur = (f, int(r[0]), r[1].strip()[:60])
        except ValueError:
            pass
        continue
    if r[2] in seen:
        continue
    seen.add(r[2])
    dd = dict(zip(hdr, r))
    sass = r[3].strip()
    if not sass:
        continue
    op = sass.split()[1] if sass.startswith("@") else sass.split()[0]
    try:
        n = int(dd["Instructions Executed"])
    except (ValueError, KeyError):
        continue
    per[cur][op] += n
    ops[op] += n
T = sum(ops.values()) or 1
print(f"total warp instructions {T} ({T / units:.0f} per unit)")
print("opcodes:", ", ".join(f"{o} {n / T * 100:.1f}%" for o, n in ops.most_common(16)))
FP = ("FFMA", "FMUL", "FFMA2", "FMUL2", "FADD", "FADD2")
lines = sorted(per.items(), key=lambda kv: -sum(n for o, n in kv[1].items() if o not in FP))
for k, c in lines[:28]:
    nf = sum(n for o, n in c.items() if o not in FP)
    print(f"{k[0]}:{k[1]:4d} nonFP {nf / units:8.1f}  {k[2]:60s} {c.most_common(2)}")
