"""GPU-side checks of the C ABI that are not stencil parity: the EXACT model's
k (Eq. 11, reading M4) against the hardware's occupancy calculator, the
kernels' register counts (Eq. 11's Rtile), and graph-cache safety of one
handle reused across tiles (the 3D progress-flag buffer growing between
captures)."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import oracle  # noqa: E402
import paper_conf_ppopp_prajapatirradg17_b200 as hhc  # noqa: E402
from oracle import model_oracle as mo  # noqa: E402
from synth import field  # noqa: E402

if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

DEV = torch.device("cuda:0")

CASES = [(hhc.HEAT2D_9PT, (32, 12, 512, 0), 384), (hhc.HEAT2D_9PT, (16, 20, 128, 0), 64),
         (hhc.HEAT2D_9PT, (8, 4, 64, 0), 32), (hhc.GRADIENT2D, (32, 12, 512, 0), 384),
         (hhc.GRADIENT2D, (8, 3, 256, 0), 128), (hhc.JACOBI2D_5PT, (4, 2, 32, 0), 16),
         (hhc.HEAT3D_7PT, (8, 8, 16, 64), 512), (hhc.HEAT3D_7PT, (4, 2, 2, 32), 64),
         (hhc.LAPLACIAN3D_27PT, (8, 6, 8, 64), 256), (hhc.LAPLACIAN3D_27PT, (2, 1, 1, 32), 8),
         (hhc.JACOBI1D_3PT, (128, 2048, 0, 0), 256), (hhc.JACOBI1D_3PT, (8, 64, 0, 0), 256),
         (hhc.BINOM1D_R3, (64, 4096, 0, 0), 256)]


@pytest.mark.parametrize("kind,tile,threads", CASES)
def test_exact_k_equals_hardware_occupancy(kind, tile, threads):
    nd = hhc.KIND_NDIMS[kind]
    smem, thr, regs = hhc.stencil_tile_resources(nd, tile, threads, kind=kind)
    assert regs > 0 and thr == threads
    assert smem == mo.smem_bytes_exact(nd, tile, hhc.KIND_RADIUS.get(kind, 1))
    props = torch.cuda.get_device_properties(0)
    hw = mo.HW(nSM=props.multi_processor_count, nV=128, MTBSM=32, RSM=65536, MSM=228 * 1024,
               Mblock=227 * 1024, L=1e-12, tau_sync=1e-9, T_sync=1e-6, C_iter=1e-9, regs_per_thread=regs,
               geometry=mo.EXACT, threads=threads)
    assert mo.k_exact(smem, threads, hw) == hhc.stencil_tile_occupancy(kind, tile, threads), (kind, tile, regs)


def test_one_handle_many_tiles_3d_flags_regrow():
    """a 3D tile needing a larger progress-flag buffer invalidates
    the cached graphs of earlier tiles; replaying tile A after B must still be
    bit-exact (stale flag pointers would hang or corrupt)."""
    dims = (40, 64, 70)
    a = field(77, dims)
    exp = oracle.run(hhc.HEAT3D_7PT, a, 9, hhc.FUSED)
    s = hhc.stencil_create(hhc.HEAT3D_7PT, dims)
    d_in = torch.from_numpy(a).to(DEV)
    outs = []
    for tile in [(4, 2, 2, 32), (2, 1, 1, 32), (4, 2, 2, 32), (2, 1, 1, 32), (4, 2, 2, 32)]:
        d_out = torch.full_like(d_in, float("nan"))
        hhc.stencil_run(s, d_in, d_out, 9, tile)
        torch.cuda.synchronize()
        outs.append(d_out.cpu().numpy())
    hhc.stencil_destroy(s)
    for o in outs:
        assert np.array_equal(o.view(np.uint32), exp.view(np.uint32))
