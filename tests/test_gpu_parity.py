"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle,
element by element on the same seeded inputs.  Bar (BASELINE.json north_star,
DESIGN.md R4/R5): bit-exact in both arithmetic modes (plain vs plain oracle,
fused vs fused oracle); fused within 1e-5 max relative error of the plain
oracle.  The full config sizes in the bench's launch configuration are in
tests/test_gpu_fullgrid.py."""
import math
import os

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import oracle  # noqa: E402
import paper_conf_ppopp_prajapatirradg17_b200 as hhc  # noqa: E402
from synth import field  # noqa: E402

if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

DEV = torch.device("cuda:0")


def gpu_run(kind, a, T, tile, mode=hhc.FUSED, threads=0, coeffs=None, env=None):
    old = {}
    for k, v in (env or {}).items():
        old[k] = os.environ.get(k)
        os.environ[k] = v
    try:
        s = hhc.stencil_create(kind, a.shape, coeffs=coeffs, mode=mode)
        d_in = torch.from_numpy(np.ascontiguousarray(a)).to(DEV)
        d_out = torch.empty_like(d_in)
        hhc.stencil_run(s, d_in, d_out, T, tile, threads)
        torch.cuda.synchronize()
        assert hhc.stencil_last_launches(s) >= 1
        res = d_out.cpu().numpy()
        hhc.stencil_destroy(s)
        return res
    finally:
        for k, v in old.items():
            if v is None:
                os.environ.pop(k, None)
            else:
                os.environ[k] = v


def assert_bits(got, exp, what=""):
    if not np.array_equal(got.view(np.uint32), exp.view(np.uint32)):
        bad = np.argwhere(got.view(np.uint32) != exp.view(np.uint32))
        i = tuple(bad[0])
        raise AssertionError(f"{what}: {len(bad)} mismatches, first at {i}: gpu {got[i]!r} oracle {exp[i]!r}")


def max_rel(got, ref):
    g, r = got.astype(np.float64), ref.astype(np.float64)
    return float(np.max(np.abs(g - r) / np.maximum(np.abs(r), 2.0 ** -10)))


TILES_2D = [(2, 1, 32), (4, 3, 32), (8, 5, 64), (6, 2, 32), (10, 7, 96), (16, 4, 128), (2, 9, 64)]
TILES_3D = [(2, 1, 1, 32), (4, 2, 3, 32), (6, 3, 4, 64), (8, 2, 2, 32), (2, 5, 6, 32), (4, 3, 2, 96), (6, 2, 3, 128)]


@pytest.mark.parametrize("kind", [hhc.JACOBI2D_5PT, hhc.HEAT2D_9PT, hhc.GRADIENT2D, hhc.LAPLACIAN2D_5PT])
@pytest.mark.parametrize("mode", [hhc.PLAIN, hhc.FUSED])
def test_parity_2d_small(kind, mode):
    rng = np.random.default_rng(kind * 10 + mode)
    for tile in TILES_2D:
        dims = (int(rng.integers(3, 90)), int(rng.integers(3, 150)))
        a = field(int(rng.integers(1, 1 << 30)), dims)
        for T in (1, 2, 5, tile[0] + 1, 2 * tile[0] + 3):
            got = gpu_run(kind, a, T, tile, mode)
            exp = oracle.run(kind, a, T, mode)
            assert_bits(got, exp, f"kind {kind} mode {mode} dims {dims} T {T} tile {tile}")


@pytest.mark.parametrize("kind", [hhc.HEAT3D_7PT, hhc.LAPLACIAN3D_27PT])
@pytest.mark.parametrize("mode", [hhc.PLAIN, hhc.FUSED])
def test_parity_3d_small(kind, mode):
    rng = np.random.default_rng(kind * 10 + mode)
    for tile in TILES_3D:
        dims = (int(rng.integers(3, 30)), int(rng.integers(3, 30)), int(rng.integers(3, 80)))
        a = field(int(rng.integers(1, 1 << 30)), dims)
        for T in (1, 3, tile[0] + 1, 2 * tile[0] + 1):
            exp = oracle.run(kind, a, T, mode)
            got = gpu_run(kind, a, T, tile, mode)
            assert_bits(got, exp, f"kind {kind} dims {dims} T {T} tile {tile}")
            got1 = gpu_run(kind, a, T, tile, mode, env={"HHC_J": "1"})      # single block per slab
            assert_bits(got1, exp, f"J=1 kind {kind} dims {dims} T {T} tile {tile}")


@pytest.mark.parametrize("threads", [0, 8, 16, 24, 64])
def test_threads_variants(threads):
    """K1 with 1-8 x-groups; K2 (3D) likewise on a grid whose rows are 16-B chunks."""
    a = field(5, (77, 133))
    tile = (6, 3, 32)
    exp = oracle.run(hhc.HEAT2D_9PT, a, 19, hhc.FUSED)
    got = gpu_run(hhc.HEAT2D_9PT, a, 19, tile, hhc.FUSED, threads=threads)
    assert_bits(got, exp, f"threads {threads}")
    b = field(15, (37, 29, 68))
    exp3 = oracle.run(hhc.HEAT3D_7PT, b, 17, hhc.FUSED)
    for tile3 in ((6, 3, 2, 32), (4, 5, 3, 64)):
        base = (tile3[3] // 4) * tile3[2]             # K2 column threads: 4 tS3 columns per tS2 line
        thr = base * max(1, threads // 8)
        if thr <= 512:
            assert_bits(gpu_run(hhc.HEAT3D_7PT, b, 17, tile3, hhc.FUSED, threads=thr), exp3, f"3D threads {thr}")


def test_T0_and_tiny_grids():
    a = field(3, (3, 3))
    assert_bits(gpu_run(hhc.HEAT2D_9PT, a, 0, (2, 1, 32)), a)
    assert_bits(gpu_run(hhc.HEAT2D_9PT, a, 4, (2, 1, 32)), oracle.run(hhc.HEAT2D_9PT, a, 4, hhc.FUSED))
    b = field(4, (3, 3, 3))
    assert_bits(gpu_run(hhc.LAPLACIAN3D_27PT, b, 3, (2, 1, 1, 32)),
                oracle.run(hhc.LAPLACIAN3D_27PT, b, 3, hhc.FUSED))
    c = field(6, (40, 5))        # tile far larger than the grid
    assert_bits(gpu_run(hhc.JACOBI2D_5PT, c, 9, (16, 30, 256)), oracle.run(hhc.JACOBI2D_5PT, c, 9, hhc.FUSED))


def test_custom_coefficients_and_c():
    a = field(8, (50, 70))
    offs, w = oracle.stencil_info(hhc.HEAT2D_9PT)
    coeffs = [float(x) * 0.9 for x in w] + [0.01]
    for mode in (hhc.PLAIN, hhc.FUSED):
        exp = oracle.run(hhc.HEAT2D_9PT, a, 11, mode, coeffs=coeffs)
        got = gpu_run(hhc.HEAT2D_9PT, a, 11, (4, 3, 32), mode, coeffs=coeffs)
        assert_bits(got, exp, f"coeffs mode {mode}")
    exp = oracle.run(hhc.GRADIENT2D, a, 7, hhc.FUSED, coeffs=[0.2])
    assert_bits(gpu_run(hhc.GRADIENT2D, a, 7, (4, 2, 32), coeffs=[0.2]), exp, "kappa")


@pytest.mark.parametrize("kind,dims,T,tile", [
    (hhc.JACOBI2D_5PT, (256, 256), 64, (8, 8, 64)),                 # C1 exactly
    (hhc.HEAT2D_9PT, (1030, 1100), 64, (16, 20, 128)),
    (hhc.GRADIENT2D, (700, 900), 40, (8, 6, 256)),
    (hhc.HEAT3D_7PT, (64, 66, 130), 20, (8, 4, 4, 32)),
    (hhc.LAPLACIAN3D_27PT, (60, 50, 70), 12, (4, 3, 4, 64)),
    (hhc.HEAT3D_7PT, (50, 60, 136), 21, (6, 4, 5, 64)),            # S3 % 4 == 0: 16-B u2-halo loads
    (hhc.LAPLACIAN3D_27PT, (41, 37, 200), 13, (8, 3, 4, 128)),
])
def test_parity_mid_size(kind, dims, T, tile):
    a = field(42, dims)
    for mode in (hhc.PLAIN, hhc.FUSED):
        exp = oracle.run(kind, a, T, mode)
        got = gpu_run(kind, a, T, tile, mode)
        assert_bits(got, exp, f"{kind} {dims} mode {mode}")
    plain = oracle.run(kind, a, T, hhc.PLAIN)
    assert max_rel(gpu_run(kind, a, T, tile, hhc.FUSED), plain) <= 1e-5


@pytest.mark.parametrize("kind,dims,T,tT,world,overlap", [
    (hhc.HEAT2D_9PT, (131, 150), 37, 8, 3, 0),
    (hhc.HEAT2D_9PT, (2 * 160 + 2, 300), 37, 8, 2, 1),
    (hhc.GRADIENT2D, (90, 77), 21, 4, 2, 0),
    (hhc.GRADIENT2D, (3 * 60 + 2, 130), 21, 4, 3, 1),
    (hhc.JACOBI2D_5PT, (4 * 40 + 2, 70), 19, 6, 4, 1),
    (hhc.HEAT3D_7PT, (40, 30, 70), 11, 4, 2, 0),
    (hhc.HEAT3D_7PT, (2 * 40 + 2, 30, 70), 13, 4, 2, 1),
    (hhc.LAPLACIAN3D_27PT, (45, 22, 40), 9, 2, 3, 0),
    (hhc.LAPLACIAN3D_27PT, (3 * 20 + 2, 22, 40), 9, 2, 3, 1),
])
def test_dist_local_virtual_ranks(kind, dims, T, tT, world, overlap):
    """The library's multi-GPU slab path (hhc_dist.cu: partition, ghost-extended
    planes, per-tile exchange, plain or overlapped edge/interior phases) with
    `world` virtual ranks of this GPU (stencil_run_dist_local; device copies in
    place of ncclSend/ncclRecv).  Every held row must equal the oracle."""
    a = field(99 + overlap, dims)
    tile = (tT, 3, 32) if len(dims) == 2 else (tT, 2, 3, 32)
    s = hhc.stencil_create(kind, dims)
    d_in = torch.from_numpy(a).to(DEV)
    d_out = torch.full_like(d_in, float("nan"))
    hhc.stencil_run_dist_local(s, world, d_in, d_out, T, tile, 0, overlap)
    assert hhc.stencil_last_launches(s) > 0
    hhc.stencil_destroy(s)
    assert_bits(d_out.cpu().numpy(), oracle.run(kind, a, T, hhc.FUSED), f"world {world} overlap {overlap}")


@pytest.mark.parametrize("kind,dims,T,tile,world,threads", [
    (hhc.HEAT2D_9PT, (300, 150), 37, (8, 3, 32), 2, 0),
    (hhc.HEAT2D_9PT, (4 * 90 + 2, 700), 45, (8, 5, 512), 4, 384),
    (hhc.GRADIENT2D, (3 * 70 + 2, 130), 21, (4, 4, 32), 3, 0),
    (hhc.JACOBI2D_5PT, (2 * 120 + 2, 300), 64, (16, 6, 256), 2, 0),
    (hhc.LAPLACIAN2D_5PT, (5 * 40 + 2, 90), 13, (6, 2, 64), 5, 0),
])
def test_hexdist_local_virtual_ranks(kind, dims, T, tile, world, threads):
    """f1: hexagons assigned to ranks by centre column, every
    point computed once, facets a neighbour stores written straight into its
    planes by the edge CTAs (stencil_run_hexdist_local, virtual ranks of one
    GPU).  The whole grid must equal the oracle bit for bit."""
    for mode in (hhc.PLAIN, hhc.FUSED):
        a = field(400 + kind + mode, dims)
        s = hhc.stencil_create(kind, dims, mode=mode)
        d_in = torch.from_numpy(a).to(DEV)
        d_out = torch.full_like(d_in, float("nan"))
        hhc.stencil_run_hexdist_local(s, world, d_in, d_out, T, tile, threads)
        n = hhc.stencil_last_launches(s)
        hhc.stencil_destroy(s)
        assert_bits(d_out.cpu().numpy(), oracle.run(kind, a, T, mode), f"hexdist world {world} mode {mode}")
        assert n > 0


@pytest.mark.parametrize("kind,dims,T,tile,threads", [
    (hhc.HEAT2D_9PT, (200, 2000), 37, (8, 6, 64), 0),
    (hhc.GRADIENT2D, (90, 3000), 21, (16, 8, 128), 64),
    (hhc.JACOBI2D_5PT, (70, 5000), 50, (32, 12, 512), 384),
])
def test_planes_2d_pipelined_blocks(kind, dims, T, tile, threads):
    """stencil_run_planes (the slab sub-problem) on a short, wide 2D domain: few
    hexagons, so each prism is split over J > 1 blocks pipelined along S2, the
    2-column face of sub-tile j2-1 handed over through global scratch after an
    acquire on its flag.  Must equal the oracle on the same domain (its outer
    rows are the fixed ring)."""
    for mode in (hhc.PLAIN, hhc.FUSED):
        a = field(500 + kind + mode, dims)
        s = hhc.stencil_create(kind, dims, mode=mode)
        p0 = torch.from_numpy(a).to(DEV)
        p1 = torch.empty_like(p0)
        for rep in range(2):                      # graph replay with the flags reset per run
            p0.copy_(torch.from_numpy(a).to(DEV))
            hhc.stencil_run_planes(s, dims[0], p0, p1, T, tile, threads)
            torch.cuda.synchronize()
            got = (p0 if T % 2 == 0 else p1).cpu().numpy()
            assert_bits(got, oracle.run(kind, a, T, mode), f"planes J>1 kind {kind} mode {mode} rep {rep}")
        hhc.stencil_destroy(s)


def test_run_host_batch_pipelined():
    """stencil_run_host_batch: independent problems from/to pinned host buffers
    with the copies overlapping the runs (two device buffer pairs); every result
    equals the oracle, 2D and 3D, n = 1..5 (buffer reuse after two steps)."""
    for kind, dims, T, tile in ((hhc.HEAT2D_9PT, (70, 130), 17, (6, 3, 32)),
                                (hhc.HEAT3D_7PT, (20, 22, 40), 7, (4, 2, 3, 32))):
        s = hhc.stencil_create(kind, dims)
        for n in (1, 2, 5):
            ins = [torch.from_numpy(field(700 + 10 * n + i, dims)).pin_memory() for i in range(n)]
            outs = [torch.empty(dims, dtype=torch.float32).pin_memory() for _ in range(n)]
            hhc.stencil_run_host_batch(s, ins, outs, T, tile)
            for i in range(n):
                assert_bits(outs[i].numpy(), oracle.run(kind, ins[i].numpy(), T, hhc.FUSED), f"batch n={n} i={i}")
        hhc.stencil_destroy(s)


def test_dist_world1_with_nccl_communicator():
    """The dlopen'ed NCCL entry points on one GPU: ncclGetUniqueId, a one-rank
    ncclCommInitRank and ncclCommDestroy through stencil_dist_*, with a slab run in
    between (world 1: no exchange) -- bit-exact against the oracle."""
    dims, T, tile = (66, 70, 40), 9, (4, 2, 3, 32)
    a = field(6, dims)
    uid = hhc.stencil_dist_get_unique_id()
    assert len(bytes(uid)) == 128
    comm = hhc.stencil_dist_init(uid, 0, 1, 0)
    s = hhc.stencil_create(hhc.HEAT3D_7PT, dims)
    d_in = torch.from_numpy(a).to(DEV)
    d_out = torch.empty_like(d_in)
    hhc.stencil_run_dist(s, comm, d_in, d_out, T, tile)
    torch.cuda.synchronize()
    hhc.stencil_destroy(s)
    hhc.stencil_dist_destroy(comm)
    assert_bits(d_out.cpu().numpy(), oracle.run(hhc.HEAT3D_7PT, a, T, hhc.FUSED), "world 1 with NCCL")


def test_dist_world1_nccl_free():
    """stencil_run_dist on a world-1 communicator (no NCCL needed): the slab is
    the whole grid."""
    dims, T, tile = (70, 90), 13, (4, 3, 32)
    a = field(5, dims)
    comm = hhc.stencil_dist_init(None, 0, 1, 0)
    s = hhc.stencil_create(hhc.HEAT2D_9PT, dims)
    d_in = torch.from_numpy(a).to(DEV)
    d_out = torch.empty_like(d_in)
    hhc.stencil_run_dist(s, comm, d_in, d_out, T, tile)
    torch.cuda.synchronize()
    hhc.stencil_destroy(s)
    hhc.stencil_dist_destroy(comm)
    assert_bits(d_out.cpu().numpy(), oracle.run(hhc.HEAT2D_9PT, a, T, hhc.FUSED), "world 1")


PAIR_TILES = [((2, 1, 256), 0), ((4, 3, 256), 64), ((8, 5, 512), 0), ((16, 4, 256), 128), ((6, 2, 768), 192),
              ((10, 7, 1024), 128), ((16, 20, 512), 256), ((12, 9, 256), 32), ((4, 2, 32), 8), ((6, 3, 96), 24),
              ((8, 6, 160), 80), ((2, 9, 64), 0)]


@pytest.mark.parametrize("kind", [hhc.JACOBI2D_5PT, hhc.HEAT2D_9PT, hhc.GRADIENT2D, hhc.LAPLACIAN2D_5PT])
@pytest.mark.parametrize("mode", [hhc.PLAIN, hhc.FUSED])
def test_parity_pair_layout(kind, mode):
    """K1 pair layout (columns q and q + tS2/2 share a register pair, swizzled
    chunks): random sizes, grids smaller than a tile, odd T, tS2 from 32 to
    1024 (non powers of two included), several x-group counts."""
    rng = np.random.default_rng(3000 + kind * 10 + mode)
    for tile, threads in PAIR_TILES:
        dims = (int(rng.integers(3, 120)), int(rng.integers(3, 1500)))
        a = field(int(rng.integers(1, 1 << 30)), dims)
        for T in (1, 2, 3, tile[0] + 1, 2 * tile[0] + 3):
            exp = oracle.run(kind, a, T, mode)
            got = gpu_run(kind, a, T, tile, mode, threads=threads)
            assert_bits(got, exp, f"pair kind {kind} mode {mode} dims {dims} T {T} tile {tile} thr {threads}")
    offs, w = oracle.stencil_info(kind) if kind != hhc.GRADIENT2D else (None, None)
    if w is not None:
        a = field(9, (70, 700))
        coeffs = [float(x) * 0.95 for x in w] + [0.003]
        exp = oracle.run(kind, a, 11, mode, coeffs=coeffs)
        assert_bits(gpu_run(kind, a, 11, (4, 3, 512), mode, coeffs=coeffs), exp, "pair coeffs")


# ---- Jacobi-1D: K0, one block per hexagon
@pytest.mark.parametrize("mode", [hhc.PLAIN, hhc.FUSED])
def test_parity_1d(mode):
    rng = np.random.default_rng(70 + mode)
    for tile in [(2, 1), (4, 3), (8, 32), (16, 100), (64, 512), (6, 2000)]:
        n = int(rng.integers(3, 5000))
        a = field(int(rng.integers(1, 1 << 30)), (n,))
        for T in (1, 2, 7, tile[0] + 1, 3 * tile[0] + 5):
            exp = oracle.run(hhc.JACOBI1D_3PT, a, T, mode)
            got = gpu_run(hhc.JACOBI1D_3PT, a, T, tile, mode)
            assert_bits(got, exp, f"1D n {n} T {T} tile {tile}")


@pytest.mark.parametrize("kind", [hhc.BINOM1D_R2, hhc.BINOM1D_R3, hhc.BINOM1D_R4])
@pytest.mark.parametrize("mode", [hhc.PLAIN, hhc.FUSED])
def test_parity_radius_r_1d(kind, mode):
    """radius-R hexagons (slope R, pitch 2 tS1 + R tT, ring of
    width R, 2R-row footprints/facets) in K0, bit-exact against the oracle on
    random sizes, tiles (grids smaller than a tile included) and T."""
    rng = np.random.default_rng(200 + 10 * kind + mode)
    R = hhc.KIND_RADIUS[kind]
    for tile in [(2, 1), (4, 3), (8, 32), (16, 100), (64, 512), (6, 2000), (32, 4096)]:
        n = int(rng.integers(2 * R + 1, 7000))
        a = field(int(rng.integers(1, 1 << 30)), (n,))
        for T in (1, 2, 7, tile[0] + 1, 3 * tile[0] + 5):
            exp = oracle.run(kind, a, T, mode)
            got = gpu_run(kind, a, T, tile, mode)
            assert_bits(got, exp, f"radius {R} n {n} T {T} tile {tile}")
    a = field(301, (50001,))
    offs, w = oracle.stencil_info(kind)
    coeffs = [float(x) * 0.97 for x in w] + [0.002]
    assert_bits(gpu_run(kind, a, 37, (8, 512), mode, coeffs=coeffs),
                oracle.run(kind, a, 37, mode, coeffs=coeffs), "radius coeffs")
    if mode == hhc.FUSED:
        plain = oracle.run(kind, a, 100, hhc.PLAIN)
        assert max_rel(gpu_run(kind, a, 100, (32, 2048), hhc.FUSED), plain) <= 1e-5


def test_parity_1d_large_and_coeffs():
    a = field(71, (1_000_003,))
    for T, tile in ((100, (32, 2048)), (257, (64, 4096))):
        assert_bits(gpu_run(hhc.JACOBI1D_3PT, a, T, tile), oracle.run(hhc.JACOBI1D_3PT, a, T, hhc.FUSED),
                    f"1D large T {T}")
    coeffs = [0.25, 0.5, 0.25, 0.001]
    for mode in (hhc.PLAIN, hhc.FUSED):
        assert_bits(gpu_run(hhc.JACOBI1D_3PT, a[:20001], 33, (8, 256), mode, coeffs=coeffs),
                    oracle.run(hhc.JACOBI1D_3PT, a[:20001], 33, mode, coeffs=coeffs), "1D coeffs")
    plain = oracle.run(hhc.JACOBI1D_3PT, a, 100, hhc.PLAIN)
    assert max_rel(gpu_run(hhc.JACOBI1D_3PT, a, 100, (32, 2048), hhc.FUSED), plain) <= 1e-5


# ---- wavefront-parallel Jacobi-1D (reading W1): K3, one block per
# parallelogram tile, one launch per wavefront; the same oracle as every other schedule
def gpu_run_wavefront(a, T, tile, mode=hhc.FUSED, coeffs=None):
    s = hhc.stencil_create(hhc.JACOBI1D_3PT, a.shape, coeffs=coeffs, mode=mode)
    d_in = torch.from_numpy(np.ascontiguousarray(a)).to(DEV)
    d_out = torch.full_like(d_in, float("nan"))
    hhc.stencil_run_wavefront(s, d_in, d_out, T, tile)
    torch.cuda.synchronize()
    nw = hhc.stencil_wavefront_info(a.shape, T, tile)[0] if T > 0 else 0
    assert hhc.stencil_last_launches(s) == (2 + nw if T > 0 else 1)
    res = d_out.cpu().numpy()
    assert np.array_equal(d_in.cpu().numpy().view(np.uint32), a.view(np.uint32))   # in untouched
    hhc.stencil_destroy(s)
    return res


@pytest.mark.parametrize("mode", [hhc.PLAIN, hhc.FUSED])
def test_parity_wavefront_1d(mode):
    rng = np.random.default_rng(90 + mode)
    for tile in [(1, 2), (2, 3), (3, 7), (8, 32), (16, 256), (5, 1000), (64, 4096)]:
        n = int(rng.integers(3, 6000))
        a = field(int(rng.integers(1, 1 << 30)), (n,))
        for T in (0, 1, 2, 7, tile[0] + 1, 3 * tile[0] + 5):
            exp = oracle.run(hhc.JACOBI1D_3PT, a, T, mode)
            got = gpu_run_wavefront(a, T, tile, mode)
            assert_bits(got, exp, f"wavefront n {n} T {T} tile {tile}")


def test_parity_wavefront_1d_large_and_coeffs():
    a = field(91, (400_003,))
    for T, tile in ((64, (16, 2048)), (37, (4, 8192)), (100, (100, 1024))):
        assert_bits(gpu_run_wavefront(a, T, tile), oracle.run(hhc.JACOBI1D_3PT, a, T, hhc.FUSED),
                    f"wavefront large T {T} tile {tile}")
    coeffs = [0.25, 0.5, 0.25, 0.001]
    for mode in (hhc.PLAIN, hhc.FUSED):
        assert_bits(gpu_run_wavefront(a[:20001], 33, (8, 256), mode, coeffs=coeffs),
                    oracle.run(hhc.JACOBI1D_3PT, a[:20001], 33, mode, coeffs=coeffs), "wavefront coeffs")
    # the two schedules of the same update agree bit for bit
    assert_bits(gpu_run_wavefront(a, 50, (10, 512)), gpu_run(hhc.JACOBI1D_3PT, a, 50, (16, 2048)), "wave vs hex")
