#!/usr/bin/env python3
"""Per-GPU-count tiles for the multi-GPU slab path, measured on ONE GPU.

For N GPUs the busiest rank (two neighbours when N >= 3) runs ceil(T/tT) time
tiles of tT steps on a ghost-extended slab of own + e*tT rows (own =
ceil((S1-2)/N), e = 2, or 1 when N = 2).  This script times exactly that work
(stencil_run_planes on a slab of those rows, min of `reps`) for candidate tiles
and reports, per N:
  * the estimated step time T_est = (n-1) t(tT) + t(T_last) (NCCL exchange not
    included: g rows per neighbour per tile, ~1-20 us over NVLink);
  * the model's M7 prediction T_G (model_predict with n_gpus = N, calibrated
    EXACT hardware parameters, plain exchange);
  * the best measured tile, the model's Eq. 31 argmin with n_gpus = N
    (model_select_tile) and its measured T_est -> the chosen-tile gap
    (BASELINE north_star: "model-selected vs exhaustive-best tile at 8 B200",
    emulated on one GPU).

    python scripts/slab_tiles.py --config C5 --gpus 2 4 8 [--out profiles/r02/slab_C5.json]
"""
from __future__ import annotations

import argparse
import json
import math
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def candidates(nd, rows, wide=False):
    if nd == 2 and wide:
        out = [((tT, tS1, tS2, 0), thr) for tT in (4, 6, 8, 10, 12, 16, 20, 24) for tS1 in (2, 3, 4, 6, 8)
               for tS2 in (256, 512) for thr in ((tS2 // 8) * g for g in (2, 3, 4, 6, 8)) if thr <= 512]
    elif nd == 2:
        out = [((tT, tS1, tS2, 0), thr) for tT in (8, 16, 24, 32) for tS1 in (4, 8, 12, 16) for tS2 in (256, 512)
               for thr in ((tS2 // 8) * g for g in (2, 3, 6)) if thr <= 384]
    else:
        out = [((tT, tS1, tS2, tS3), thr) for tT in (4, 6, 8) for tS1 in (2, 4, 6, 8) for tS2 in (4, 8, 16)
               for tS3 in (32, 64) for thr in ((tS3 // 4) * tS2 * g for g in (1, 2)) if thr <= 512]
    return [(t, thr) for t, thr in out if 2 * t[1] + t[0] <= rows]


def main():
    import torch

    import bench
    import paper_conf_ppopp_prajapatirradg17_b200 as hhc
    from paper_conf_ppopp_prajapatirradg17_b200 import tune
    from synth import CONFIG_SEEDS, field

    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C5")
    ap.add_argument("--gpus", type=int, nargs="+", default=[2, 4, 8])
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--budget", type=float, default=900.0)
    ap.add_argument("--out", default=None)
    ap.add_argument("--wide", action="store_true", help="2D: a denser candidate set (small hexagons, up to 512 threads)")
    args = ap.parse_args()
    cfg = bench.CONFIGS[args.config]
    kind, dims, T = cfg["kind"], cfg["dims"], cfg["T"]
    nd = len(dims)
    cal = tune.load_cal()
    res = {"config": args.config, "per_gpus": {}}
    t_start = time.time()
    for N in args.gpus:
        own = -(-(dims[0] - 2) // N)
        e = 2 if N >= 3 else 1
        pts = []

        def measure(tile, thr):
            tT = tile[0]
            rows = own + e * tT + 2
            h = hhc.stencil_create(kind, (rows,) + tuple(dims[1:]))
            a = torch.from_numpy(field(CONFIG_SEEDS[args.config], (rows,) + tuple(dims[1:]))).cuda()
            p0, p1 = a.clone(), torch.empty_like(a)
            n = -(-T // tT)
            Tl = T - (n - 1) * tT
            tt = {}
            for Tt in sorted({tT, Tl}):
                best = math.inf
                for _ in range(args.reps + 1):
                    p0.copy_(a)
                    s, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    s.record()
                    hhc.stencil_run_planes(h, rows, p0, p1, Tt, tile, thr)
                    e1.record()
                    e1.synchronize()
                    best = min(best, s.elapsed_time(e1) * 1e-3)
                tt[Tt] = best
            hhc.stencil_destroy(h)
            return (n - 1) * tt[tT] + tt[Tl]

        for tile, thr in candidates(nd, own + 2 * 32, args.wide):
            if time.time() - t_start > args.budget:
                break
            try:
                te = measure(tile, thr)
            except hhc.StencilError:
                continue
            hw = tune.b200_hw(cal, kind, hhc.EXACT, thr, tile=tile)
            hw.n_gpus, hw.link_bytes_per_s, hw.link_latency_s = N, 7.7e11, 1e-5
            pts.append({"tile": list(tile), "threads": thr, "t_est": te,
                        "model_TG": hhc.model_predict(kind, dims, T, tile, hw)})
        best = min(pts, key=lambda p: p["t_est"])
        hw = tune.b200_hw(cal, kind, hhc.EXACT)
        hw.n_gpus, hw.link_bytes_per_s, hw.link_latency_s = N, 7.7e11, 1e-5
        entry = {"own_rows": own, "n_points": len(pts), "best_measured": best, "points": pts}
        try:
            bt, bthr, cands = hhc.model_select_tile(kind, dims, T, hw, 0.10)
            te = measure(bt, bthr)
            entry["model_argmin"] = {"tile": list(bt), "threads": bthr, "t_est": te,
                                     "model_TG": hhc.model_predict(kind, dims, T, bt, hw),
                                     "gap_vs_best_measured": te / best["t_est"] - 1.0, "n_within_10pct": len(cands)}
        except hhc.StencilError as err:
            entry["model_argmin"] = {"error": str(err)}
        res["per_gpus"][str(N)] = entry
        print(json.dumps({"N": N, "best": best, "model_argmin": entry["model_argmin"]}), flush=True)
    out = args.out or os.path.join(ROOT, "profiles", "r02", f"slab_{args.config}.json")
    os.makedirs(os.path.dirname(out), exist_ok=True)
    with open(out, "w") as f:
        json.dump(res, f, indent=1)


if __name__ == "__main__":
    main()
