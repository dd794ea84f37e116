"""Experiment: time a list of tiles for one config in one process.
usage: python scripts/exp_tiles.py C4 8,4,8,64:256 ...   (threads 0 = library rule)
T may be reduced with HHC_EXP_T (updates/s stays comparable)."""
import os, sys, torch
sys.path.insert(0, '.')
import bench
import paper_conf_ppopp_prajapatirradg17_b200 as hhc
from paper_conf_ppopp_prajapatirradg17_b200.tune import time_run
cfg = bench.CONFIGS[sys.argv[1]]
T = int(os.environ.get("HHC_EXP_T", cfg["T"]))
h = hhc.stencil_create(cfg["kind"], cfg["dims"])
a = torch.rand(*cfg["dims"], device='cuda'); b = torch.empty_like(a)
n = hhc.updates(cfg["dims"], T)
for spec in sys.argv[2:]:
    t, thr = spec.split(':')
    tile = tuple(int(x) for x in t.split(','))
    tile = tile + (0,) * (4 - len(tile))
    try:
        te = time_run(h, a, b, T, tile, int(thr), reps=2)
        print(f"{spec:22s} {te*1e3:9.2f} ms {n/te/1e9:9.1f} G/s", flush=True)
    except Exception as e:
        print(f"{spec:22s} ERR {e}", flush=True)
