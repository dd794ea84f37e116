"""f1 across PROCESSES: each rank a separate process with its own
CUDA context, planes exported/opened as CUDA IPC handles (peer-mapped), K1's
facet stores going straight into the neighbour's planes, row-by-row device-side
flag handshakes (stencil_run_hexdist).  The ranks share this GPU (NCCL would
refuse two ranks on one device; CUDA IPC does not), so the whole cross-process
path -- export, open, peer stores, acquire/release flags -- runs here exactly
as across GPUs.  torch.distributed (gloo) only carries the 192-byte handles."""
import os
import socket

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _rank(rank, world, port, kind, dims, T, tile, threads, runs, outdir):
    import torch.distributed as dist

    import paper_conf_ppopp_prajapatirradg17_b200 as hhc
    from synth import field
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    torch.cuda.set_device(0)
    b0, b1, xl, xh, hl, hh = hhc.stencil_hexdist_partition(dims[0], rank, world, tile)
    h = hhc.stencil_create(kind, dims)
    obj, mine = hhc.stencil_hexdist_create(h, rank, world, tile)
    allh = [None] * world
    dist.all_gather_object(allh, mine)
    hhc.stencil_hexdist_connect(h, obj, allh[rank - 1] if rank > 0 else None,
                                allh[rank + 1] if rank < world - 1 else None)
    dist.barrier()
    d_in = torch.from_numpy(field(777, dims, row_start=xl, nrows=xh - xl)).cuda()
    d_out = torch.full((hh - hl,) + tuple(dims[1:]), float("nan"), device="cuda")
    for _ in range(runs):                      # repeated runs: the epoch handshake across runs
        hhc.stencil_run_hexdist(h, obj, d_in, d_out, T, threads)
    torch.cuda.synchronize()
    np.save(os.path.join(outdir, f"r{rank}.npy"), d_out.cpu().numpy())
    np.save(os.path.join(outdir, f"rows{rank}.npy"), np.array([hl, hh]))
    dist.barrier()
    hhc.stencil_hexdist_destroy(obj)
    hhc.stencil_destroy(h)
    dist.destroy_process_group()


@pytest.mark.parametrize("kind,dims,T,tile,world,threads,runs", [
    (2, (2 * 100 + 2, 300), 29, (8, 5, 64), 2, 0, 2),
    (3, (3 * 80 + 2, 200), 17, (4, 6, 32), 3, 0, 1),
    (1, (4 * 60 + 2, 530), 40, (8, 4, 512), 4, 384, 2),
])
def test_hexdist_ipc_processes(tmp_path, kind, dims, T, tile, world, threads, runs):
    import torch.multiprocessing as mp

    import oracle
    from synth import field
    port = _free_port()
    mp.spawn(_rank, args=(world, port, kind, dims, T, tile, threads, runs, str(tmp_path)), nprocs=world, join=True)
    exp = oracle.run(kind, field(777, dims), T, oracle.FUSED)
    got = np.full_like(exp, np.nan)
    for r in range(world):
        lo, hi = np.load(tmp_path / f"rows{r}.npy")
        got[lo:hi] = np.load(tmp_path / f"r{r}.npy")
    assert np.array_equal(got.view(np.uint32), exp.view(np.uint32))
