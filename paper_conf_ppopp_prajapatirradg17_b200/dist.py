"""Multi-GPU slab decomposition of the HHC path (BASELINE.json
north_star -- not in the paper).

The interior S1 rows are split into `world` contiguous slabs of
own = ceil((S1-2)/world) rows.  Every time tile of tT steps:

  1. ghost exchange: each rank sends its first / last g = tT owned rows to
     rank -/+ 1 and receives its top / bottom ghost rows (torch.distributed
     P2P: NCCL over NVLink on GPUs, gloo in the CPU tests);
  2. the rank runs tT steps of HHC on its ghost-extended slab with the
     slab's outermost rows held fixed (stencil_run_planes, all compute in the
     CUDA kernels).  After tT steps every owned row is exact, because the
     dependence cone of tT steps of a radius-1 stencil reaches tT rows.

The level-0 plane of the next tile is the output plane of this one (tT even),
so no copy is made between tiles.  All collectives are point to point; there
is no reduction on the data path.  Orchestration only: the per-tile stepper is
a callable so the CPU tests can run the same driver with the oracle as stepper.
"""
from __future__ import annotations

import math
import os
import time
from dataclasses import dataclass


@dataclass
class Slab:
    rank: int
    world: int
    S1: int
    own: int        # interior rows per rank (last rank may own fewer)
    r0: int         # first owned interior row
    r1: int         # one past the last owned interior row
    e0: int         # first row of the ghost-extended slab
    e1: int         # one past the last row of the extended slab
    g: int          # ghost depth (= tT)

    @property
    def rows(self) -> int:
        return self.e1 - self.e0

    @property
    def held(self):
        """Rows of the global grid the rank's in/out slab holds: the owned
        rows plus the physical ring row on the edge ranks."""
        lo = self.r0 - (1 if self.rank == 0 else 0)
        hi = self.r1 + (1 if self.rank == self.world - 1 else 0)
        return lo, hi


def partition(S1: int, world: int, rank: int, g: int) -> Slab:
    interior = S1 - 2
    own = -(-interior // world)
    r0 = 1 + rank * own
    r1 = min(1 + (rank + 1) * own, S1 - 1)
    if r1 <= r0:
        raise ValueError(f"rank {rank} owns no rows (S1={S1}, world={world})")
    if world > 1 and own < g:
        raise ValueError(f"slab of {own} rows is thinner than the ghost depth {g}: use a smaller tT")
    if world > 1 and r1 - r0 < g and rank < world - 1:
        raise ValueError("slab thinner than the ghost depth")
    e0 = max(0, r0 - g)
    e1 = min(S1, r1 + g)
    return Slab(rank, world, S1, own, r0, r1, e0, e1, g)


def exchange(slab: Slab, plane, xp_dist):
    """Fill the ghost rows of `plane` (the extended slab, rows e0..e1) from the
    neighbours' owned rows.  `xp_dist` is torch.distributed."""
    import torch
    ops = []
    g = slab.g
    lo = slab.r0 - slab.e0          # local index of the first owned row
    hi = slab.r1 - slab.e0          # local index one past the last owned row
    if slab.rank > 0:
        up_send = plane[lo:lo + g]
        up_recv = plane[lo - g:lo]
        ops.append(xp_dist.P2POp(xp_dist.isend, up_send.contiguous(), slab.rank - 1))
        ops.append(xp_dist.P2POp(xp_dist.irecv, up_recv, slab.rank - 1))
    if slab.rank < slab.world - 1:
        dn_send = plane[hi - g:hi]
        dn_recv = plane[hi:hi + g]
        ops.append(xp_dist.P2POp(xp_dist.isend, dn_send.contiguous(), slab.rank + 1))
        ops.append(xp_dist.P2POp(xp_dist.irecv, dn_recv, slab.rank + 1))
    if ops:
        for r in xp_dist.batch_isend_irecv(ops):
            r.wait()
    return torch


def run_slabs(slab: Slab, plane0, plane1, T: int, tT: int, stepper, xp_dist):
    """Drive the time tiles.  plane0 holds level 0 of the extended slab (ring and
    ghosts included); stepper(plane0, plane1, Tt) runs Tt steps leaving the
    result in plane0 (Tt even) or plane1 (Tt odd).  Returns the plane holding A_T."""
    done = 0
    cur = plane0
    while done < T:
        Tt = min(tT, T - done)
        if slab.world > 1:
            exchange(slab, cur, xp_dist)
        out = stepper(cur, plane1 if cur is plane0 else plane0, Tt)
        cur = out
        done += Tt
    return cur


def run_slabs_overlap(slab: Slab, plane0, plane1, T: int, tT: int, stepper_int, stepper_edge, xp_dist,
                      streams=None):
    """The time-tile loop with the exchange overlapped (SURVEY §8(e) "Overlap").

    Per tile: the two edge sub-slabs -- 3g rows around each neighbour side, fresh
    ghosts included -- run first (stepper_edge, second stream) and their exact
    owned rows [lo, lo+g) / [hi-g, hi) are sent to the neighbours at once; the
    interior sub-slab (the owned rows alone, whose edge rows act as a fixed ring
    for the tile) needs no ghosts and runs concurrently (stepper_int, first
    stream).  After tT <= g steps the interior run is exact on [lo+g, hi-g), the
    edge runs on the g rows next to each side (dependence cone of tT rows), so
    the tile's result is the interior plane with the edge rows and the received
    ghosts written in.  Redundant work: 3g rows per neighbour side per tile.

    `streams` = (s1, s2) torch.cuda streams, or None (CPU: sequential).  Falls
    back to run_slabs when a slab is thinner than 2g rows."""
    import torch
    g = slab.g
    lo, hi = slab.r0 - slab.e0, slab.r1 - slab.e0
    up, dn = slab.rank > 0, slab.rank < slab.world - 1
    if not (up or dn) or hi - lo < 2 * g:
        return run_slabs(slab, plane0, plane1, T, tT, stepper_int, xp_dist)
    A, B = (lo if up else 0), (hi if dn else slab.rows)
    tail = tuple(plane0.shape[1:])

    def buf(n):
        return torch.empty((n,) + tail, dtype=plane0.dtype, device=plane0.device)

    e_up = (lo - g, lo + 2 * g) if up else None          # local rows of the edge sub-slabs
    e_dn = (hi - 2 * g, hi + g) if dn else None
    t_bufs = (buf(3 * g), buf(3 * g)) if up else None
    b_bufs = (buf(3 * g), buf(3 * g)) if dn else None
    r_up = buf(g) if up else None
    r_dn = buf(g) if dn else None
    s1, s2 = streams if streams is not None else (None, None)

    def on(st):
        return torch.cuda.stream(st) if st is not None else _Null()

    exchange(slab, plane0, xp_dist)                      # ghosts of tile 0 (blocking)
    cur, oth = plane0, plane1
    done = 0
    while done < T:
        Tt = min(tT, T - done)
        last = done + Tt >= T
        with on(s1):                                     # edge inputs taken before the interior overwrites cur
            if up:
                t_bufs[0].copy_(cur[e_up[0]:e_up[1]])
            if dn:
                b_bufs[0].copy_(cur[e_dn[0]:e_dn[1]])
        if s2 is not None:
            s2.wait_stream(s1)
        works = []
        with on(s2):
            te = stepper_edge(t_bufs[0], t_bufs[1], Tt) if up else None
            be = stepper_edge(b_bufs[0], b_bufs[1], Tt) if dn else None
            if not last:
                ops = []
                if up:
                    ops.append(xp_dist.P2POp(xp_dist.isend, te[g:2 * g], slab.rank - 1))
                    ops.append(xp_dist.P2POp(xp_dist.irecv, r_up, slab.rank - 1))
                if dn:
                    ops.append(xp_dist.P2POp(xp_dist.isend, be[g:2 * g], slab.rank + 1))
                    ops.append(xp_dist.P2POp(xp_dist.irecv, r_dn, slab.rank + 1))
                works = xp_dist.batch_isend_irecv(ops)
        with on(s1):
            stepper_int(cur[A:B], oth[A:B], Tt)           # overlaps the exchange
            res = cur if Tt % 2 == 0 else oth
            if s2 is not None:
                s1.wait_stream(s2)
            for w in works:
                w.wait()
            if up:
                res[lo:lo + g].copy_(te[g:2 * g])
                if not last:
                    res[lo - g:lo].copy_(r_up)
            if dn:
                res[hi - g:hi].copy_(be[g:2 * g])
                if not last:
                    res[hi:hi + g].copy_(r_dn)
        cur, oth = res, (plane1 if res is plane0 else plane0)
        done += Tt
    return cur


class _Null:
    def __enter__(self):
        return self

    def __exit__(self, *a):
        return False


def gpu_stepper(handle, tile, threads, stream=None, counter=None):
    """Per-tile stepper on the GPU (stencil_run_planes).  `counter`, a one-element
    list, accumulates the kernel launches the library reports."""
    import paper_conf_ppopp_prajapatirradg17_b200 as hhc

    def step(p0, p1, Tt):
        hhc.stencil_run_planes(handle, p0.shape[0], p0, p1, Tt, tile, threads, stream)
        if counter is not None:
            counter[0] += hhc.stencil_last_launches(handle)
        return p0 if Tt % 2 == 0 else p1
    return step


def bench_main(args, cfg, cfgname, configs):
    """bench.py under torchrun: strong scaling of the config across ranks."""
    import json

    import torch
    import torch.distributed as dist

    import paper_conf_ppopp_prajapatirradg17_b200 as hhc
    from synth import CONFIG_SEEDS, field

    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", str(args.gpus)))
    local = int(os.environ.get("LOCAL_RANK", str(rank)))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    dist.init_process_group("nccl", device_id=dev)
    tile = tuple(int(x) for x in args.tile.split(",")) if args.tile else cfg["tile"]
    tile = tile + (0,) * (4 - len(tile))
    threads = cfg["threads"] if args.threads is None else args.threads
    dims, T, kind = cfg["dims"], cfg["T"], cfg["kind"]
    strong = not bool(getattr(args, "weak", False))
    if not strong:
        # weak scaling (default): every rank owns a slab of the config's interior
        # rows, the global grid is world times taller; ghost exchange as usual
        dims = ((dims[0] - 2) * world + 2,) + tuple(dims[1:])
    tT = tile[0]
    slab = partition(dims[0], world, rank, tT)
    ext_dims = (slab.rows,) + tuple(dims[1:])
    host = field(CONFIG_SEEDS[cfgname], dims, row_start=slab.e0, nrows=slab.rows)
    init = torch.from_numpy(host).to(dev)
    p0 = torch.empty_like(init)
    p1 = torch.empty_like(init)
    mode = hhc.FUSED if args.mode == "fused" else hhc.PLAIN
    h = hhc.stencil_create(kind, ext_dims, mode=mode)
    stream = torch.cuda.current_stream()
    launches = [0]
    step = gpu_stepper(h, tile, threads, stream, launches)
    overlap = not getattr(args, "no_overlap", False)
    if overlap:
        # edge sub-slabs on a second stream with their own handle (3D progress flags)
        side = torch.cuda.Stream(device=dev)
        h_edge = hhc.stencil_create(kind, ext_dims, mode=mode)
        step_edge = gpu_stepper(h_edge, tile, threads, side, launches)

    def drive(a, b):
        if overlap:
            return run_slabs_overlap(slab, a, b, T, tT, step, step_edge, dist, (stream, side))
        return run_slabs(slab, a, b, T, tT, step, dist)

    def one():
        p0.copy_(init)
        return drive(p0, p1)

    for _ in range(args.warmup):
        one()
    torch.cuda.synchronize()
    dist.barrier()
    import bench
    sampler = bench.ClockSampler(local) if rank == 0 else None
    if sampler:
        sampler.start()
        time.sleep(0.3)
    launches[0] = 0
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for _ in range(args.steps):
        one()
    e1.record(stream)
    torch.cuda.synchronize()
    dist.barrier()
    clocks = sampler.stop() if sampler else None
    t = torch.tensor([e0.elapsed_time(e1) * 1e-3, float(launches[0])], device=dev)
    tmax = t.clone()
    dist.all_reduce(tmax, op=dist.ReduceOp.MAX)
    tsum = t.clone()
    dist.all_reduce(tsum, op=dist.ReduceOp.SUM)
    dt = float(tmax[0].item())
    # copies p0 <- init per step (one kernel each) plus the HHC launches of every rank
    n_launch = int(tsum[1].item()) + world * args.steps

    # e2e through the public API: pinned host slab -> device, the run, owned rows -> host
    e2e = None
    if not args.no_e2e:
        h_in = torch.from_numpy(host).pin_memory()
        lo, hi = slab.held
        h_out = torch.empty((hi - lo,) + tuple(dims[1:]), dtype=torch.float32).pin_memory()

        def one_e2e():
            p0.copy_(h_in, non_blocking=True)
            out = drive(p0, p1)
            h_out.copy_(out[lo - slab.e0:hi - slab.e0], non_blocking=True)
            torch.cuda.synchronize()

        one_e2e()
        dist.barrier()
        t0 = time.perf_counter()
        for _ in range(args.steps):
            one_e2e()
        et = torch.tensor([time.perf_counter() - t0], device=dev)
        dist.all_reduce(et, op=dist.ReduceOp.MAX)
        nb = torch.tensor([float(host.nbytes), float(h_out.numel() * 4)], device=dev)
        dist.all_reduce(nb, op=dist.ReduceOp.SUM)
        e2e = {"value": hhc.updates(dims, T) * args.steps / float(et.item()) / 1e9, "unit": "GStencil-updates/s",
               "h2d_bytes_per_step": int(nb[0].item()), "d2h_bytes_per_step": int(nb[1].item())}
    n_upd = hhc.updates(dims, T)
    if rank == 0:
        line = {"metric": "GStencil-updates/s", "value": round(n_upd * args.steps / dt / 1e9, 3),
                "unit": "GStencil-updates/s", "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
                "ms_per_step": round(dt / args.steps * 1e3, 3), "higher_is_better": True, "scaling": "strong" if strong else "weak",
                "vs_baseline": None, "dtype": "f32", "data": "synthetic",
                "config": {"workload": cfgname + ": " + cfg["desc"] + (
                               "" if strong else f", weak-scaled: {world} slabs of the config's rows, global grid "
                                                 f"{'x'.join(map(str, dims))}"), "tile": list(tile), "threads": threads,
                           "parallelism": f"{world} S1 slabs, ghost depth {tT}, NCCL P2P every time tile"
                                          + (", exchange overlapped with the interior sub-slab (edge sub-slabs "
                                             "first on a second stream)" if overlap else ""),
                           "l2": "inputs larger than L2"},
                "roofline": bench.alu_roofline(kind, n_upd * args.steps / dt / world, bench.load_peaks(),
                                               traffic=None,
                                               kernel="hex2d_kernel" if len(dims) == 2 else "hex3d_kernel",
                                               achieved_basis="updates per GPU per second of the whole step "
                                                              "(max over ranks; redundancy and exchange "
                                                              "included)"),
                "e2e": e2e, "clocks": clocks, "gpu_launches": n_launch}
        print(json.dumps(line))
    hhc.stencil_destroy(h)
    if overlap:
        hhc.stencil_destroy(h_edge)
    dist.destroy_process_group()
    return 0
