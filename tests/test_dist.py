"""Multi-process (gloo, CPU) tests of the slab decomposition driver
(paper_conf_ppopp_prajapatirradg17_b200/dist.py): partition, ghost
exchange and the time-tile loop, with the CPU oracle as the per-tile stepper.
The gathered owned rows must equal the single-domain oracle bit for bit."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import slab_reference as hdist
from synth import field


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, kind, dims, T, tT, seed, outdir, overlap=False):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    slab = hdist.partition(dims[0], world, rank, tT)
    init = field(seed, dims, row_start=slab.e0, nrows=slab.rows)
    p0 = torch.from_numpy(init.copy())
    p1 = torch.empty_like(p0)

    def step(a, b, Tt):
        res = torch.from_numpy(oracle.run(kind, a.numpy(), Tt, oracle.FUSED))
        if Tt % 2 == 0:
            a.copy_(res)
            return a
        b.copy_(res)
        return b

    if overlap:
        out = hdist.run_slabs_overlap(slab, p0, p1, T, tT, step, step, dist)
    else:
        out = hdist.run_slabs(slab, p0, p1, T, tT, step, dist)
    lo, hi = slab.held
    np.save(os.path.join(outdir, f"r{rank}.npy"), out[lo - slab.e0:hi - slab.e0].numpy())
    np.save(os.path.join(outdir, f"rows{rank}.npy"), np.array([lo, hi]))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world,kind,dims,T,tT", [
    (2, oracle.HEAT2D_9PT, (41, 37), 13, 4),
    (3, oracle.GRADIENT2D, (50, 29), 9, 2),
    (2, oracle.JACOBI2D_5PT, (34, 40), 8, 8),
    (2, oracle.HEAT3D_7PT, (22, 9, 11), 7, 2),
    (3, oracle.LAPLACIAN3D_27PT, (26, 8, 7), 6, 4),
])
def test_slab_decomposition_matches_oracle(tmp_path, world, kind, dims, T, tT):
    port = _free_port()
    mp.spawn(_worker, args=(world, port, kind, dims, T, tT, 77, str(tmp_path)), nprocs=world, join=True)
    full = oracle.run(kind, field(77, dims), T, oracle.FUSED)
    got = np.empty_like(full)
    covered = np.zeros(dims[0], bool)
    for r in range(world):
        lo, hi = np.load(tmp_path / f"rows{r}.npy")
        got[lo:hi] = np.load(tmp_path / f"r{r}.npy")
        assert not covered[lo:hi].any()
        covered[lo:hi] = True
    assert covered.all()
    assert np.array_equal(got.view(np.uint32), full.view(np.uint32))


@pytest.mark.parametrize("world,kind,dims,T,tT", [
    (2, oracle.HEAT2D_9PT, (41, 37), 13, 4),          # T not a multiple of tT: odd last tile
    (3, oracle.GRADIENT2D, (62, 29), 9, 2),
    (4, oracle.JACOBI2D_5PT, (70, 23), 17, 4),
    (2, oracle.HEAT3D_7PT, (30, 9, 11), 7, 2),
    (3, oracle.LAPLACIAN3D_27PT, (38, 8, 7), 6, 4),
    (3, oracle.HEAT2D_9PT, (20, 16), 8, 4),           # slabs thinner than 2g: falls back to run_slabs
])
def test_overlapped_exchange_matches_oracle(tmp_path, world, kind, dims, T, tT):
    """§8(e) overlap: edge sub-slabs first (their owned rows are what is sent),
    interior sub-slab concurrently, result assembled per tile -- bit-exact."""
    port = _free_port()
    mp.spawn(_worker, args=(world, port, kind, dims, T, tT, 78, str(tmp_path), True), nprocs=world, join=True)
    full = oracle.run(kind, field(78, dims), T, oracle.FUSED)
    got = np.empty_like(full)
    for r in range(world):
        lo, hi = np.load(tmp_path / f"rows{r}.npy")
        got[lo:hi] = np.load(tmp_path / f"r{r}.npy")
    assert np.array_equal(got.view(np.uint32), full.view(np.uint32))


def test_partition_rules():
    s = hdist.partition(8194, 8, 0, 16)
    assert (s.r0, s.e0, s.held) == (1, 0, (0, s.r1))
    s7 = hdist.partition(8194, 8, 7, 16)
    assert s7.r1 == 8193 and s7.e1 == 8194 and s7.held[1] == 8194
    with pytest.raises(ValueError):
        hdist.partition(40, 8, 0, 16)            # slabs thinner than the ghost depth


def test_product_partition_matches_reference():
    """The library's slab geometry (stencil_dist_partition, used by
    stencil_run_dist) equals the algorithm reference tested above."""
    import paper_conf_ppopp_prajapatirradg17_b200 as hhc
    for S1 in (20, 41, 70, 1000, 8194, 16386):
        for world in (1, 2, 3, 4, 7, 8):
            for g in (2, 4, 8, 16, 32):
                for rank in range(world):
                    try:
                        s = hdist.partition(S1, world, rank, g)
                    except ValueError:
                        with pytest.raises(hhc.StencilError):
                            hhc.stencil_dist_partition(S1, rank, world, g)
                        continue
                    assert hhc.stencil_dist_partition(S1, rank, world, g) == (s.r0, s.r1, s.e0, s.e1) + s.held


def test_hexdist_partition_rules():
    """f1 partition (host only): owned rows tile [1, S1-1) exactly, stored rows
    extend H = tS1/2 + tT/2 + 3 on each side (clipped to the grid), the held
    rows add the physical ring on the edge ranks, and slabs thinner than 2H are
    rejected (a hexagon would reach two ranks away)."""
    import paper_conf_ppopp_prajapatirradg17_b200 as hhc
    for S1, world, tile in [(362, 4, (8, 5, 512)), (1000, 3, (16, 12, 64)), (8194, 8, (32, 12, 512))]:
        H = tile[1] // 2 + tile[0] // 2 + 3
        prev_b1 = 1
        for r in range(world):
            b0, b1, xl, xh, hl, hh = hhc.stencil_hexdist_partition(S1, r, world, tile)
            assert b0 == prev_b1 and b1 > b0
            assert xl == max(0, b0 - H) and xh == min(S1, b1 + H)
            assert hl == (0 if r == 0 else b0) and hh == (S1 if r == world - 1 else b1)
            prev_b1 = b1
        assert prev_b1 == S1 - 1
    with pytest.raises(hhc.StencilError):
        hhc.stencil_hexdist_partition(100, 0, 8, (16, 12, 64))
