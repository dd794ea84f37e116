"""Multi-GPU bootstrap and bench orchestration of the slab path (
BASELINE.json north_star -- not in the paper).

The data path is the library's: stencil_run_dist (csrc/hhc_dist.cu) partitions
the S1 rows, exchanges the g = tT ghost rows with ncclSend/ncclRecv every time
tile and runs the HHC rows on the ghost-extended slab.  torch.distributed is
used only to start the ranks and to broadcast the NCCL unique id (plus the
barrier and max-over-ranks timing of the bench).  The exchange variant (plain
or overlapped) comes from the model's reading M7 (model_predict with
n_gpus = N), the tile per GPU count from the config's table, see `choose_tile`.
"""
from __future__ import annotations

import os
import time


def init_comm(rank: int, world: int, device: int, torch_dist):
    """NCCL communicator of the library: rank 0's unique id is broadcast over the
    process group (the only thing torch.distributed carries)."""
    import paper_conf_ppopp_prajapatirradg17_b200 as hhc
    uid = [hhc.stencil_dist_get_unique_id() if rank == 0 and world > 1 else None]
    if world > 1:
        torch_dist.broadcast_object_list(uid, src=0)
    return hhc.stencil_dist_init(uid[0], rank, world, device)


def slab_rows(S1: int, rank: int, world: int, g: int):
    """(held_lo, held_hi): the global rows this rank's in/out slab holds."""
    import paper_conf_ppopp_prajapatirradg17_b200 as hhc
    part = hhc.stencil_dist_partition(S1, rank, world, g)
    return part[4], part[5]


def choose_tile(cfg: dict, world: int, hw_json: str | None = None):
    """Tile, threads and exchange variant for `world` GPUs: the config's tile
    table (bench.CONFIGS[..]["tiles_by_gpus"], measured on the slab sizes) when
    it has an entry, else the config tile; the exchange variant by the M7 model
    (plain vs overlapped) with the committed B200 calibration."""
    tile = tuple(cfg.get("tiles_by_gpus", {}).get(world, cfg["tile"]))
    threads = cfg.get("threads_by_gpus", {}).get(world, cfg["threads"])
    overlap = model_overlap_choice(cfg, world, tile, hw_json) if world > 1 else 0
    return tile, threads, overlap


def model_overlap_choice(cfg: dict, world: int, tile, hw_json: str | None = None) -> int:
    """1 if M7 predicts the overlapped exchange faster than the plain one."""
    import json

    import paper_conf_ppopp_prajapatirradg17_b200 as hhc
    from paper_conf_ppopp_prajapatirradg17_b200 import tune
    path = hw_json or os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "profiles",
                                   "hw_params_b200.json")
    cal = json.load(open(path))
    hw = tune.b200_hw(cal, cfg["kind"], hhc.EXACT)
    hw.n_gpus, hw.link_bytes_per_s, hw.link_latency_s = world, 7.7e11, 1e-5
    t = []
    for ov in (0, 1):
        hw.dist_overlap = ov
        t.append(hhc.model_predict(cfg["kind"], cfg["dims"], cfg["T"], tile, hw))
    return 1 if t[1] < t[0] else 0


def bench_main(args, cfg, cfgname, configs):
    """bench.py under torchrun: the config's grid split over the ranks (strong
    scaling; --weak: one config-sized slab per rank)."""
    import json

    import torch
    import torch.distributed as dist

    import bench
    import paper_conf_ppopp_prajapatirradg17_b200 as hhc
    from synth import CONFIG_SEEDS, field

    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", str(args.gpus)))
    local = int(os.environ.get("LOCAL_RANK", str(rank)))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    dist.init_process_group("nccl", device_id=dev)
    dims, T, kind = cfg["dims"], cfg["T"], cfg["kind"]
    strong = not bool(getattr(args, "weak", False))
    if not strong:
        dims = ((dims[0] - 2) * world + 2,) + tuple(dims[1:])
    tile, threads, overlap = choose_tile(cfg, world)
    if args.tile:
        tile = tuple(int(x) for x in args.tile.split(","))
    tile = tuple(tile) + (0,) * (4 - len(tile))
    if args.threads is not None:
        threads = args.threads
    if getattr(args, "no_overlap", False):
        overlap = 0
    mode = hhc.FUSED if args.mode == "fused" else hhc.PLAIN
    h = hhc.stencil_create(kind, dims, mode=mode)
    stream = torch.cuda.current_stream()
    launches = [0]
    hexdist = getattr(args, "exchange", "slab") == "hexdist"
    if hexdist:
        # f1: hexagons by centre column, facets peer-stored into the neighbours' planes
        # (CUDA IPC handles carried by torch.distributed; no NCCL on the data path)
        comm = None
        b0, b1, xl, xh, lo, hi = hhc.stencil_hexdist_partition(dims[0], rank, world, tile)
        obj, mine = hhc.stencil_hexdist_create(h, rank, world, tile)
        allh = [None] * world
        dist.all_gather_object(allh, mine)
        hhc.stencil_hexdist_connect(h, obj, allh[rank - 1] if rank > 0 else None,
                                    allh[rank + 1] if rank < world - 1 else None)
        dist.barrier()
        stored = torch.from_numpy(field(CONFIG_SEEDS[cfgname], dims, row_start=xl, nrows=xh - xl)).to(dev)
        host = field(CONFIG_SEEDS[cfgname], dims, row_start=lo, nrows=hi - lo)
        d_in = stored
        d_out = torch.empty((hi - lo,) + tuple(dims[1:]), dtype=torch.float32, device=dev)
        overlap = 0

        def one():
            hhc.stencil_run_hexdist(h, obj, d_in, d_out, T, threads, stream)
            launches[0] += hhc.stencil_last_launches(h)
    else:
        comm = init_comm(rank, world, local, dist)
        hhc.stencil_dist_set_overlap(comm, overlap)
        lo, hi = slab_rows(dims[0], rank, world, tile[0])
        host = field(CONFIG_SEEDS[cfgname], dims, row_start=lo, nrows=hi - lo)
        d_in = torch.from_numpy(host).to(dev)
        d_out = torch.empty_like(d_in)

        def one():
            hhc.stencil_run_dist(h, comm, d_in, d_out, T, tile, threads, stream)
            launches[0] += hhc.stencil_last_launches(h)

    for _ in range(args.warmup):
        one()
    torch.cuda.synchronize()
    dist.barrier()
    sampler = bench.ClockSampler(local) if rank == 0 else None
    if sampler:
        sampler.start()
        time.sleep(0.3)
    launches[0] = 0
    torch.cuda.synchronize()
    dist.barrier()
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
    n_launch = int(tsum[1].item())

    # e2e through the public API: pinned host slab -> device, the run, the slab -> host
    e2e = None
    if not args.no_e2e:
        h_in = torch.from_numpy(d_in.cpu().numpy()).pin_memory()
        h_out = torch.empty(tuple(d_out.shape), dtype=torch.float32).pin_memory()

        def one_e2e():
            d_in.copy_(h_in, non_blocking=True)
            one()
            h_out.copy_(d_out, non_blocking=True)
            torch.cuda.synchronize()

        one_e2e()
        dist.barrier()
        t0 = time.perf_counter()
        for _ in range(args.steps):
            one_e2e()
        et = torch.tensor([time.perf_counter() - t0], device=dev)
        dist.all_reduce(et, op=dist.ReduceOp.MAX)
        nb = torch.tensor([float(h_in.numel() * 4), float(h_out.numel() * 4)], device=dev)
        dist.all_reduce(nb, op=dist.ReduceOp.SUM)
        e2e = {"value": hhc.updates(dims, T) * args.steps / float(et.item()) / 1e9, "unit": "GStencil-updates/s",
               "h2d_bytes_per_step": int(nb[0].item()), "d2h_bytes_per_step": int(nb[1].item())}
    n_upd = hhc.updates(dims, T)
    if rank == 0:
        line = {"metric": "GStencil-updates/s", "value": round(n_upd * args.steps / dt / 1e9, 3),
                "unit": "GStencil-updates/s", "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
                "ms_per_step": round(dt / args.steps * 1e3, 3), "higher_is_better": True,
                "scaling": "strong" if strong else "weak", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
                "config": {"workload": cfgname + ": " + cfg["desc"] + (
                               "" if strong else f", weak-scaled: {world} slabs of the config's rows, global grid "
                                                 f"{'x'.join(map(str, dims))}"), "tile": list(tile), "threads": threads,
                           "parallelism": (f"{world} ranks, hexagons by centre column, facets peer-stored over "
                                           f"NVLink into the neighbours' planes (stencil_run_hexdist, f1)" if hexdist else
                                           f"{world} S1 slabs, ghost depth {tile[0]}, ncclSend/ncclRecv every time "
                                           f"tile (stencil_run_dist, "
                                           + ("edge sub-slabs overlapped with the interior)" if overlap
                                              else "exchange then the ghost-extended slab)")),
                           "l2": "inputs larger than L2"},
                "roofline": bench.alu_roofline(kind, n_upd * args.steps / dt / world, bench.load_peaks(),
                                               traffic=None,
                                               kernel="hex2d_kernel" if len(dims) == 2 else "hex3d_kernel",
                                               achieved_basis="updates per GPU per second of the whole step "
                                                              "(max over ranks; redundancy and exchange "
                                                              "included)"),
                "e2e": e2e, "clocks": clocks, "gpu_launches": n_launch}
        print(json.dumps(line))
    torch.cuda.synchronize()
    dist.barrier()
    if hexdist:
        hhc.stencil_hexdist_destroy(obj)
    else:
        hhc.stencil_dist_destroy(comm)
    hhc.stencil_destroy(h)
    dist.destroy_process_group()
    return 0
