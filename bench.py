#!/usr/bin/env python3
"""bench.py -- GStencil-updates/s of the HHC stencil path on B200.

A "step" is one pass of the whole hot path (plan, buffer
setup, every row of hexagons) over one synthetic input: T time steps of the
config's stencil on its full grid.  Default workload: C3, Gradient-2D fp32,
16384^2, T = 512 -- the BASELINE.json config quoted at 1/2/4/8 GPUs, so the
N = 1 line and the scaling run measure the same problem.  --config C1..C5
(and the extension configs X1, W1) select the others.  The tile is the one
listed in CONFIGS (model_select_tile + the measured sweep).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config C3] [--impl reference]

Under torchrun (N > 1) the config's grid is slab-decomposed along S1 across
the ranks (strong scaling, the BASELINE 1/2/4/8 experiment) with a ghost
exchange every time tile; --weak gives every rank a config-sized slab instead.
Rank 0 prints the line; times are the max over ranks of device (CUDA-event)
time.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

CONFIGS = {
    "C1": dict(kind=1, dims=(256, 256), T=64, tile=(12, 1, 512, 0), threads=384,
               desc="Jacobi-2D 5-point fp32, 256x256, T=64"),
    "C2": dict(kind=2, dims=(8192, 8192), T=1024, tile=(32, 12, 512, 0), threads=384,
               desc="Heat-2D 9-point fp32, 8192x8192, T=1024"),
    # tiles_by_gpus: the tile per GPU count under torchrun, the best measured on one GPU for
    # the slab each rank holds (scripts/slab_tiles.py -> profiles/r02/slab_C{3,4,5}.json)
    "C3": dict(kind=3, dims=(16384, 16384), T=512, tile=(32, 12, 512, 0), threads=384,
               tiles_by_gpus={2: (32, 12, 512, 0), 4: (24, 3, 512, 0), 8: (12, 3, 512, 0)},
               threads_by_gpus={4: 512, 8: 512},
               desc="Gradient-2D fp32, 16384x16384, T=512"),
    "C4": dict(kind=4, dims=(512, 512, 512), T=256, tile=(8, 8, 16, 64), threads=512,
               tiles_by_gpus={2: (8, 6, 16, 64), 4: (8, 2, 16, 64), 8: (6, 2, 16, 64)},
               desc="Heat-3D 7-point fp32, 512^3, T=256"),
    "C5": dict(kind=5, dims=(768, 768, 768), T=128, tile=(8, 10, 14, 64), threads=448,
               tiles_by_gpus={8: (8, 2, 16, 64)}, threads_by_gpus={8: 512},
               desc="Laplacian-3D 27-point fp32, 768^3, T=128"),
    # SURVEY §8(f) f2 (not a BASELINE.json config): the paper's 1D derivation case
    "X1": dict(kind=7, dims=(1 << 26,), T=1024, tile=(128, 2048), threads=256,
               desc="Jacobi-1D 3-point fp32, 2^26 points, T=1024 (extension f2)"),
    # SURVEY §8(f) f3 (not a BASELINE.json config): the wavefront-parallel schedule
    "W1": dict(kind=7, dims=((1 << 22) + 2,), T=1024, tile=(4, 8192), threads=256, schedule="wavefront",
               desc="Jacobi-1D 3-point fp32, 2^22 interior points, T=1024, wavefront schedule (extension f3)"),
    # SURVEY §8(f) f4 (not a BASELINE.json config): a higher-order (radius-2) stencil under HHC
    "X2": dict(kind=8, dims=(1 << 26,), T=1024, tile=(64, 2048), threads=256,
               desc="Binomial-1D radius-2 5-point fp32, 2^26 points, T=1024 (extension f4)"),
}
DEFAULT_CONFIG = "C3"

# n_fp32 of SURVEY §8(d): FP32-pipe instructions per update (one FFMA/FMUL/FADD
# lane operation each; a packed FFMA2 counts 2).  Linear kinds: |N| (1 FMUL +
# |N|-1 FFMA of the canonical fused expression).  Gradient-2D: counted in the
# kernel's SASS (FP32-pipe lane ops of the IEEE sqrt and division sequences
# included, MUFU excluded), scripts/count_fp32.py -> profiles/r02/n_fp32_gradient.txt.
N_FP32 = {1: 5, 2: 9, 3: 24.4, 4: 7, 5: 27, 6: 5, 7: 3, 8: 5, 9: 7, 10: 9}
N_FP32_SOURCE = {3: "SASS count of the Gradient-2D row step (profiles/r02/n_fp32_gradient.txt)"}

METRIC = "GStencil-updates/s"


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(p) as f:
            return json.load(f)
    except OSError:
        return {}


def p_fma(peaks) -> float:
    """P_fma of SURVEY §8(d): FP32-pipe lane instructions per second = 148 SMs x
    128 FP32 lanes x max SM clock (MEASURED_PEAKS.json sm_max_mhz); measured on
    this B200 at 120-126 FMA/clk/SM (scripts/ubench/ffma2.cu, profiles/r02/probe)."""
    mhz = float(peaks.get("sm_max_mhz", 1965.0))
    return 148 * 128 * mhz * 1e6


def alu_roofline(kind: int, upd_per_s: float, peaks: dict, **extra) -> dict:
    """roofline = P_fma / n_fp32 updates/s; frac = achieved / that."""
    n = N_FP32[kind]
    peak = p_fma(peaks) / n / 1e9
    ach = upd_per_s / 1e9
    d = {"bound": "alu", "achieved": round(ach, 3), "peak": round(peak, 2), "unit": "GStencil-updates/s",
         "frac": round(ach / peak, 4), "n_fp32": n,
         "peak_basis": "P_fma / n_fp32: 148 SM x 128 FP32 lanes x sm_max_mhz (MEASURED_PEAKS.json) "
                       "FP32-pipe instr/s over n_fp32 per update (SURVEY 8(d))"}
    if kind in N_FP32_SOURCE:
        d["n_fp32_source"] = N_FP32_SOURCE[kind]
    d.update(extra)
    return d


class ClockSampler:
    """nvidia-smi clocks/throttle reasons DURING the timed region (B200_PROFILING.md)."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int = 0):
        self.index = index
        self.proc = None
        self.path = os.path.join("/tmp", f"hhc_clocks_{os.getpid()}.csv")

    def start(self):
        try:
            self.f = open(self.path, "w")
            self.proc = subprocess.Popen(["nvidia-smi", f"--id={self.index}", f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=self.f, stderr=subprocess.DEVNULL)
        except OSError:
            self.proc = None

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.25)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except subprocess.TimeoutExpired:
            self.proc.kill()
        self.f.close()
        rows = []
        for line in open(self.path):
            parts = [x.strip() for x in line.split(",")]
            if len(parts) >= 9:
                rows.append(parts)
        os.unlink(self.path)
        if not rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["no samples"]}
        sm = sorted(float(r[1]) for r in rows if r[1].replace(".", "").isdigit())
        mx = max(float(r[2]) for r in rows if r[2].replace(".", "").isdigit())
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in rows for i in range(4) if r[5 + i].lower() == "active"})
        load = [s for s in sm if s > 0.5 * mx] or sm
        return {"sm_mhz": load[len(load) // 2], "sm_max_mhz": mx, "reasons": reasons,
                "samples": len(rows)}


def ncu_traffic(cfg: str):
    """dram bytes per launch of the dominant kernel from the committed ncu summary."""
    for name in sorted(os.listdir(os.path.join(ROOT, "profiles")), reverse=True) if os.path.isdir(
            os.path.join(ROOT, "profiles")) else []:
        if name.startswith("ncu_summary") and name.endswith(".json"):
            try:
                d = json.load(open(os.path.join(ROOT, "profiles", name)))
            except (OSError, ValueError):
                continue
            if cfg in d and d[cfg].get("dram_bytes_per_launch"):
                return d[cfg]["dram_bytes_per_launch"]
    return None


def hhc_updates(dims, T, kind):
    """Interior updates T * prod(S_d - 2R), R the kind's ring width (1; 2-4 for f4)."""
    R = {8: 2, 9: 3, 10: 4}.get(int(kind), 1)
    return int(T) * math.prod(int(d) - 2 * R for d in dims)


def cpu_oracle_sample(cfg: dict, seconds: float = 10.0, nthreads: int = 0):
    """The oracle as it stands (plain mode, all host cores) on a bounded sample
    of the workload: the full grid for T_s < T steps, T_s sized to ~`seconds`."""
    import oracle
    from synth import CONFIG_SEEDS, field
    name = [k for k, v in CONFIGS.items() if v is cfg][0]
    a = field(CONFIG_SEEDS[name], cfg["dims"])
    n_int = hhc_updates(cfg["dims"], 1, cfg["kind"])
    oracle.run(cfg["kind"], a, 1, oracle.PLAIN, nthreads=nthreads)        # warm (threads, first touch)
    t0 = time.perf_counter()
    oracle.run(cfg["kind"], a, 2, oracle.PLAIN, nthreads=nthreads)
    one = max((time.perf_counter() - t0) / 2, 1e-4)
    Ts = int(max(1, min(cfg["T"], seconds / one)))
    t0 = time.perf_counter()
    oracle.run(cfg["kind"], a, Ts, oracle.PLAIN, nthreads=nthreads)
    dt = time.perf_counter() - t0
    if dt < 0.5 * seconds and Ts < cfg["T"]:           # the 2-step estimate was pessimistic: resize once
        Ts = int(max(1, min(cfg["T"], Ts * seconds / max(dt, 1e-3))))
        t0 = time.perf_counter()
        oracle.run(cfg["kind"], a, Ts, oracle.PLAIN, nthreads=nthreads)
        dt = time.perf_counter() - t0
    cores = nthreads or oracle.max_threads()
    return {"value": n_int * Ts / dt / 1e9, "unit": METRIC, "cores": cores, "kind": "oracle",
            "sample": f"full {'x'.join(map(str, cfg['dims']))} grid, {Ts} of {cfg['T']} steps, plain mode, "
                      f"{dt:.1f} s"}


def run_reference(args, cfg, cfgname):
    """--impl reference: the CPU oracle (the tier's reference arm) on host cores."""
    import oracle
    from synth import CONFIG_SEEDS, field
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    a = field(CONFIG_SEEDS[cfgname], cfg["dims"])
    n_int = hhc_updates(cfg["dims"], 1, cfg["kind"])
    t0 = time.perf_counter()
    oracle.run(cfg["kind"], a, 1, oracle.PLAIN)
    one = max(time.perf_counter() - t0, 1e-4)
    budget = 150.0 / max(1, args.steps + args.warmup)      # whole run within a few minutes
    Ts = int(max(1, min(cfg["T"], budget / one)))
    for _ in range(args.warmup):
        oracle.run(cfg["kind"], a, Ts, oracle.PLAIN)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        oracle.run(cfg["kind"], a, Ts, oracle.PLAIN)
    dt = time.perf_counter() - t0
    v = n_int * Ts * args.steps / dt / 1e9
    cores = oracle.max_threads()
    sample = f"full {'x'.join(map(str, cfg['dims']))} grid, {Ts} of {cfg['T']} steps per step, plain mode"
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": METRIC, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": dt / args.steps * 1e3,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f32",
            "data": "synthetic", "config": {"workload": cfgname + ": " + cfg["desc"]},
            "cpu_baseline": {"value": v, "unit": METRIC, "cores": cores, "kind": "oracle", "sample": sample},
            "e2e": {"value": v, "unit": METRIC, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line))
    return 0


def main(argv=None):
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default=DEFAULT_CONFIG, choices=sorted(CONFIGS))
    ap.add_argument("--impl", default="hhc", choices=["hhc", "reference"])
    ap.add_argument("--tile", default=None, help="override tile t,s1,s2[,s3]")
    ap.add_argument("--threads", type=int, default=None)
    ap.add_argument("--mode", default="fused", choices=["fused", "plain"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-overlap", action="store_true",
                    help="N>1: exchange, then the whole ghost-extended slab (no overlap)")
    ap.add_argument("--exchange", default="slab", choices=["slab", "hexdist"],
                    help="N > 1: NCCL ghost-row slabs (default) or the non-redundant hexagon-aligned decomposition "
                         "with peer-mapped facet stores (f1, 2D configs)")
    ap.add_argument("--weak", action="store_true",
                    help="N > 1: one config-sized slab per rank (default: strong scaling, the config's grid split "
                         "over the ranks)")
    args = ap.parse_args(argv)
    cfg = CONFIGS[args.config]
    if args.impl == "reference":
        return run_reference(args, cfg, args.config)
    world = int(os.environ.get("WORLD_SIZE", "1"))
    if world > 1 or args.gpus > 1:
        from paper_conf_ppopp_prajapatirradg17_b200 import dist
        return dist.bench_main(args, cfg, args.config, CONFIGS)
    return bench_single(args, cfg, args.config)


def bench_single(args, cfg, cfgname):
    import numpy as np
    import torch

    import paper_conf_ppopp_prajapatirradg17_b200 as hhc
    from synth import CONFIG_SEEDS, field

    assert args.warmup >= 3 or os.environ.get("HHC_BENCH_ALLOW_SHORT"), "W >= 3 warm-up steps required"
    torch.cuda.set_device(0)
    dev = torch.device("cuda:0")
    tile = tuple(int(x) for x in args.tile.split(",")) if args.tile else cfg["tile"]
    tile = tile + (0,) * (4 - len(tile))
    threads = cfg["threads"] if args.threads is None else args.threads
    mode = hhc.FUSED if args.mode == "fused" else hhc.PLAIN
    dims, T, kind = cfg["dims"], cfg["T"], cfg["kind"]
    n_upd = hhc.updates(dims, T, kind)

    host = field(CONFIG_SEEDS[cfgname], dims)
    h_in = torch.from_numpy(host).pin_memory()
    d_in = h_in.to(dev, non_blocking=False)
    d_out = torch.empty_like(d_in)
    s = hhc.stencil_create(kind, dims, mode=mode)
    stream = torch.cuda.current_stream()

    wave = cfg.get("schedule") == "wavefront"

    def run(a, b):
        if wave:
            hhc.stencil_run_wavefront(s, a, b, T, tile, stream)
        else:
            hhc.stencil_run(s, a, b, T, tile, threads, stream)

    for _ in range(args.warmup):
        run(d_in, d_out)
    torch.cuda.synchronize()
    launches_per_step = hhc.stencil_last_launches(s)

    sampler = ClockSampler(0)
    sampler.start()
    time.sleep(0.3)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record(stream)
    for _ in range(args.steps):
        run(d_in, d_out)
    e1.record(stream)
    torch.cuda.synchronize()
    clocks = sampler.stop()
    dt = e0.elapsed_time(e1) * 1e-3
    ms_per_step = dt / args.steps * 1e3
    value = n_upd * args.steps / dt / 1e9

    # dominant kernel: per-launch device time of the HHC rows (events on the launching stream)
    if wave:
        # the wavefront launches are one CUDA graph with the two set-up copies (16 MB each, < 1 % of the
        # step): the kernel time is the step time
        ksec, klaunch = dt / args.steps, launches_per_step - 2
    else:
        ksec, klaunch = hhc.stencil_profile(s, d_in, d_out, T, tile, threads, stream)
    traffic = ncu_traffic(cfgname)
    roofline = alu_roofline(kind, n_upd / ksec, load_peaks(), traffic=traffic,
                            kernel="wave1d_kernel" if wave else {1: "hex1d_kernel", 2: "hex2d_kernel",
                                                                 3: "hex3d_kernel"}[len(dims)],
                            kernel_share_of_step=round(ksec / (dt / args.steps), 4),
                            kernel_launches_per_step=klaunch,
                            achieved_basis="updates per step / summed CUDA-event time of the HHC row launches")

    e2e = None
    if not args.no_e2e:
        h_out = torch.empty_like(h_in).pin_memory()

        def run_host():
            if wave:     # pinned host -> device, run, device -> host, synchronise
                d_in.copy_(h_in, non_blocking=True)
                run(d_in, d_out)
                h_out.copy_(d_out, non_blocking=True)
                torch.cuda.synchronize()
            else:
                hhc.stencil_run_host(s, h_in, h_out, T, tile, threads, stream)

        if wave:
            run_host()
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            for _ in range(args.steps):
                run_host()
            et = time.perf_counter() - t0
        else:
            # every step is one problem from/to pinned host memory through the public call;
            # stencil_run_host_batch overlaps step i+1's H2D and step i-1's D2H with step i's run
            hhc.stencil_run_host_batch(s, [h_in] * 2, [h_out] * 2, T, tile, threads, stream)
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            hhc.stencil_run_host_batch(s, [h_in] * args.steps, [h_out] * args.steps, T, tile, threads, stream)
            et = time.perf_counter() - t0
        nbytes = host.nbytes
        e2e = {"value": n_upd * args.steps / et / 1e9, "unit": METRIC, "h2d_bytes_per_step": nbytes,
               "d2h_bytes_per_step": nbytes,
               "api": "per step: pinned H2D, stencil_run_wavefront, D2H" if wave else
                      "stencil_run_host_batch (pinned host in/out every step; step i+1's H2D and step i-1's "
                      "D2H overlap step i's run on the library's copy streams)"}
        # the e2e result must be the same numbers
        assert torch.equal(h_out, d_out.cpu()), "e2e result differs from device result"

    cpu = None if args.no_cpu_baseline else cpu_oracle_sample(cfg)
    line = {
        "metric": METRIC, "value": round(value, 3), "unit": METRIC, "n_gpus": 1, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": round(ms_per_step, 3), "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
        "config": {"workload": cfgname + ": " + cfg["desc"], "tile": list(tile), "threads": threads,
                   "mode": args.mode, "updates_per_step": n_upd,
                   "l2": "inputs larger than L2 (plane %d MB > 126 MB)" % (host.nbytes >> 20)
                   if host.nbytes > 126e6 else ("planes of %d MB stay in L2, not flushed (extension config: "
                                                "each wavefront re-reads rows the previous launch wrote)"
                                                % (host.nbytes >> 20) if wave
                                                else "inputs smaller than L2 (launch-bound config)"),
                   "parallelism": "1 GPU, one CTA per parallelogram tile, one launch per wavefront" if wave
                   else "1 GPU, one CTA per hexagonal prism"},
        "roofline": roofline, "cpu_baseline": cpu, "e2e": e2e, "clocks": clocks,
        "gpu_launches": launches_per_step * args.steps,
    }
    print(json.dumps(line))
    hhc.stencil_destroy(s)
    return 0


if __name__ == "__main__":
    sys.exit(main())
