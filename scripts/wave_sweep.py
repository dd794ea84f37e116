"""Wavefront-parallel Jacobi-1D on one B200: tile sweep of the
wavefront schedule on workload W1 (2^22 interior points, T = 1024), measured
time (CUDA events, min of 3 after a warm run) next to model_predict_wavefront
(PAPER and EXACT, the committed B200 calibration of kind 7), RMSE of
(Talg - Texec)/Texec over all points and the near-best ones (within 25 %),
the model argmin's measured gap to the best swept tile, and the hexagonal
schedule's time on the same workload for comparison.

    python scripts/wave_sweep.py [--out gpurun_out/wave/sweep_W1.json]
"""
import argparse
import json
import math
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_ppopp_prajapatirradg17_b200 as hhc  # noqa: E402
from paper_conf_ppopp_prajapatirradg17_b200 import tune  # noqa: E402
from synth import field  # noqa: E402


def timed(fn, reps=3):
    s = torch.cuda.current_stream()
    fn(s)
    torch.cuda.synchronize()
    best = math.inf
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(s)
        fn(s)
        b.record(s)
        b.synchronize()
        best = min(best, a.elapsed_time(b) * 1e-3)
    return best


def summarise(res):
    pts = res["points"]
    best = min(pts, key=lambda p: p["texec"])
    res["best"] = best
    for key in ("talg_paper", "talg_exact"):
        ra, rn, nn = tune.stats(pts, key)
        am = min((p for p in pts if math.isfinite(p[key])), key=lambda p: p[key])
        res[key] = {"rmse_all": ra, "rmse_near": rn, "n_near": nn, "argmin": am["tile"],
                    "argmin_gap": am["texec"] / best["texec"] - 1}


def rescore(path, out):
    with open(path) as f:
        res = json.load(f)
    n, T = res["n"], res["T"]
    cal = tune.load_cal()
    hwp = tune.b200_hw(cal, hhc.JACOBI1D_3PT, hhc.PAPER)
    hwe = tune.b200_hw(cal, hhc.JACOBI1D_3PT, hhc.EXACT)
    for p in res["points"]:
        p["talg_paper"] = hhc.model_predict_wavefront((n,), T, tuple(p["tile"]), hwp)
        p["talg_exact"] = hhc.model_predict_wavefront((n,), T, tuple(p["tile"]), hwe)
    summarise(res)
    os.makedirs(os.path.dirname(os.path.abspath(out)), exist_ok=True)
    with open(out, "w") as f:
        json.dump(res, f, indent=1)
    print(json.dumps({k: res[k] for k in ("best", "talg_paper", "talg_exact", "hex_best")}))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "wave", "sweep_W1.json"))
    ap.add_argument("--n", type=int, default=1 << 22)
    ap.add_argument("--T", type=int, default=1024)
    ap.add_argument("--rescore", help="recompute the model columns and statistics of an existing sweep JSON "
                    "with the current library (CPU only) and write it to --out")
    args = ap.parse_args()
    if args.rescore:
        return rescore(args.rescore, args.out)
    n, T = args.n + 2, args.T
    a = field(5, (n,))
    d_in = torch.from_numpy(a).cuda()
    d_out = torch.empty_like(d_in)
    h = hhc.stencil_create(hhc.JACOBI1D_3PT, (n,))
    cal = tune.load_cal()
    hwp = tune.b200_hw(cal, hhc.JACOBI1D_3PT, hhc.PAPER)
    hwe = tune.b200_hw(cal, hhc.JACOBI1D_3PT, hhc.EXACT)
    pts = []
    for tT in (2, 4, 8, 16, 32, 64, 128):
        for tS in (256, 512, 1024, 2048, 4096, 8192):
            t = timed(lambda s: hhc.stencil_run_wavefront(h, d_in, d_out, T, (tT, tS), s))
            nw, nt, mx = hhc.stencil_wavefront_info((n,), T, (tT, tS))
            p = {"tile": [tT, tS], "texec": t, "gups": (n - 2) * T / t / 1e9, "wavefronts": nw, "tiles": nt,
                 "max_width": mx,
                 "talg_paper": hhc.model_predict_wavefront((n,), T, (tT, tS), hwp),
                 "talg_exact": hhc.model_predict_wavefront((n,), T, (tT, tS), hwe)}
            pts.append(p)
            print(json.dumps(p), flush=True)
    res = {"workload": f"W1: Jacobi-1D 3-point fp32, {n - 2} interior points, T={T}, wavefront schedule",
           "n": n, "T": T, "points": pts}
    summarise(res)
    # Eq. 31 over the whole search space (reading W3): the selected tile measured, gap to the best swept
    for key, hw in (("select_paper", hwp), ("select_exact", hwe)):
        sel, cands = hhc.model_select_wavefront_tile((n,), T, hw, 0.10)
        t = timed(lambda s: hhc.stencil_run_wavefront(h, d_in, d_out, T, sel, s))
        res[key] = {"tile": list(sel), "texec": t, "gups": (n - 2) * T / t / 1e9,
                    "gap_vs_best_swept": t / res["best"]["texec"] - 1, "n_candidates_10pct": len(cands)}
    # the hexagonal schedule on the same workload (K0), a few tiles, best kept
    hexpts = []
    for tile in ((64, 2048), (128, 2048), (256, 2048), (128, 4064), (256, 4064)):
        t = timed(lambda s: hhc.stencil_run(h, d_in, d_out, T, tile, 0, s))
        hexpts.append({"tile": list(tile), "texec": t, "gups": (n - 2) * T / t / 1e9})
    res["hex"] = hexpts
    res["hex_best"] = min(hexpts, key=lambda p: p["texec"])
    os.makedirs(os.path.dirname(args.out), exist_ok=True)
    with open(args.out, "w") as f:
        json.dump(res, f, indent=1)
    print(json.dumps({k: res.get(k) for k in ("best", "talg_paper", "talg_exact", "select_paper", "select_exact",
                                                "hex_best")}))


if __name__ == "__main__":
    main()
