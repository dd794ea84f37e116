"""GPU parity at the launch configurations bench.py times (tile AND threads of
bench.CONFIGS), over the WHOLE grid: the CUDA path through the C ABI against
the CPU oracle element by element (bit-exact, fused mode = the bench's mode),
at the BASELINE.json sizes for C1-C4 and at >= 400^3 for C5; plain mode and
fused-vs-plain (<= 1e-5, reading R5) at mid sizes with the same tiles and
threads; and closed forms whose decay over T steps is far above their
tolerance, so an identity kernel fails them (asserted)."""
import math

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import bench  # noqa: E402
import oracle  # noqa: E402
import paper_conf_ppopp_prajapatirradg17_b200 as hhc  # noqa: E402
from synth import CONFIG_SEEDS, field  # noqa: E402

if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

DEV = torch.device("cuda:0")


def gpu_run(kind, a, T, tile, threads, mode=hhc.FUSED):
    s = hhc.stencil_create(kind, a.shape, mode=mode)
    try:
        d_in = torch.from_numpy(np.ascontiguousarray(a)).to(DEV)
        d_out = torch.full_like(d_in, float("nan"))
        hhc.stencil_run(s, d_in, d_out, T, tile, threads)
        torch.cuda.synchronize()
        res = d_out.cpu().numpy()
        assert np.array_equal(d_in.cpu().numpy().view(np.uint32), np.asarray(a).view(np.uint32))
        return res
    finally:
        hhc.stencil_destroy(s)


def assert_bits(got, exp, what):
    g, e = got.view(np.uint32), exp.view(np.uint32)
    if not np.array_equal(g, e):
        bad = np.argwhere(g != e)
        i = tuple(bad[0])
        raise AssertionError(f"{what}: {len(bad)} of {got.size} differ, first at {i}: gpu {got[i]!r} "
                             f"oracle {exp[i]!r}")


def launch(cfg):
    c = bench.CONFIGS[cfg]
    return c["kind"], tuple(c["tile"]), c["threads"]


# (config, dims, T): the BASELINE sizes, C5 reduced (the oracle needs ~2 min at 768^3)
WHOLE = [("C1", (256, 256), 64), ("C2", (8192, 8192), 1024), ("C3", (16384, 16384), 512),
         ("C4", (512, 512, 512), 256), ("C5", (400, 400, 400), 128)]


@pytest.mark.parametrize("cfg,dims,T", WHOLE)
def test_whole_grid_bench_launch(cfg, dims, T):
    kind, tile, threads = launch(cfg)
    a = field(CONFIG_SEEDS[cfg], dims)
    got = gpu_run(kind, a, T, tile, threads)
    exp = oracle.run(kind, a, T, hhc.FUSED)
    assert_bits(got, exp, f"{cfg} whole grid {dims} T {T} tile {tile} x {threads}")


MID = [("C2", (2050, 4100), 96), ("C3", (2048, 4096), 96), ("C4", (202, 210, 230), 40),
       ("C5", (200, 204, 206), 30)]


@pytest.mark.parametrize("cfg,dims,T", MID)
def test_mid_grid_bench_launch_plain_and_fused(cfg, dims, T):
    """Both arithmetic modes bit-exact at the bench tile/threads on a ragged
    mid-size grid (several tiles and sub-tiles, partial last ones), and the
    fused path within 1e-5 of the plain oracle."""
    kind, tile, threads = launch(cfg)
    a = field(CONFIG_SEEDS[cfg] + 100, dims)
    plain = oracle.run(kind, a, T, hhc.PLAIN)
    assert_bits(gpu_run(kind, a, T, tile, threads, hhc.PLAIN), plain, f"{cfg} plain")
    fused = gpu_run(kind, a, T, tile, threads, hhc.FUSED)
    assert_bits(fused, oracle.run(kind, a, T, hhc.FUSED), f"{cfg} fused")
    g, r = fused.astype(np.float64), plain.astype(np.float64)
    assert float(np.max(np.abs(g - r) / np.maximum(np.abs(r), 2.0 ** -10))) <= 1e-5


def sine_mode(kind, dims, T):
    """Separable sine mode u0 = prod_d sin(pi p_d i_d/(S_d-1)) (ring exactly 0)
    with the smallest p = (q, .., q) whose closed-form decay lambda^T is <= 0.6:
    lambda(theta) = sum_a w_a prod_d cos(theta_d a_d)."""
    offs, w = oracle.stencil_info(kind)
    nd = len(dims)
    for q in range(1, 400):
        th = np.array([math.pi * q / (dims[d] - 1) for d in range(nd)])
        lam = sum(float(wj) * np.prod(np.cos(th * np.asarray(o[:nd]))) for o, wj in zip(offs, w))
        if abs(lam) ** T <= 0.6:
            break
    sines = []
    for d in range(nd):
        sv = np.sin(th[d] * np.arange(dims[d]))
        sv[0] = sv[-1] = 0.0
        sines.append(sv)
    return lam, sines, len(w)


@pytest.mark.parametrize("cfg", ["C2", "C4", "C5"])
def test_closed_form_decay_bench_launch(cfg):
    """Whole grid at the BASELINE size: u_T = lambda^T u0 within
    (4 T |N| + 2) 2^-24; lambda^T <= 0.6, so the identity map (and any kernel
    that skips levels) is far outside the tolerance -- asserted below."""
    kind, tile, threads = launch(cfg)
    c = bench.CONFIGS[cfg]
    dims, T = c["dims"], c["T"]
    lam, sines, npts = sine_mode(kind, dims, T)
    nd = len(dims)
    rest = sines[1][:, None] * sines[2][None, :] if nd == 3 else sines[1]
    u0 = (sines[0].reshape([-1] + [1] * (nd - 1)) * rest[None]).astype(np.float32)
    got = gpu_run(kind, u0, T, tile, threads)
    tol = (4 * T * npts + 2) * 2.0 ** -24
    err_id = 0.0
    for x0 in range(0, dims[0], 64):                  # slab-wise, bounded host memory
        ex = (lam ** T) * sines[0][x0:x0 + 64].reshape([-1] + [1] * (nd - 1)) * rest[None]
        assert np.max(np.abs(got[x0:x0 + 64].astype(np.float64) - ex)) <= tol, (cfg, lam, x0)
        err_id = max(err_id, float(np.max(np.abs(u0[x0:x0 + 64].astype(np.float64) - ex))))
    assert err_id > 50 * tol, (cfg, err_id, tol)     # the identity kernel would fail this test


@pytest.mark.parametrize("cfg", ["C2", "C3", "C4"])
def test_affine_fixed_point_bench_launch(cfg):
    """Symmetric weights summing to 1 (dyadic) and the Gradient body map an
    affine field with short-mantissa values to itself exactly."""
    kind, tile, threads = launch(cfg)
    c = bench.CONFIGS[cfg]
    dims, T = c["dims"], c["T"]
    nd = len(dims)
    aff = np.ones(dims, np.float32)
    for d, k in zip(range(nd), (1.0, 2.0, 3.0)):
        aff += (k * np.arange(dims[d], dtype=np.float32)).reshape([-1 if e == d else 1 for e in range(nd)])
    assert np.array_equal(gpu_run(kind, aff, T, tile, threads), aff), cfg


@pytest.mark.parametrize("cfg,n", [("C3", 2), ("C3", 4), ("C3", 8), ("C4", 2), ("C4", 4), ("C4", 8), ("C5", 8)])
def test_dist_bench_tiles_virtual_ranks(cfg, n):
    """The tile and threads bench.py uses under torchrun at n GPUs (tiles_by_gpus),
    through the library's slab path with n virtual ranks of this GPU
    (stencil_run_dist_local: the per-rank phases of stencil_run_dist, device copies
    in place of NCCL) on a reduced grid with the same per-rank row count ratio:
    every held row bit-exact against the oracle."""
    import paper_conf_ppopp_prajapatirradg17_b200.dist as dist
    c = bench.CONFIGS[cfg]
    tile, threads, overlap = dist.choose_tile(c, n)
    kind = c["kind"]
    rows = max(3 * tile[0], 24) * n + 2
    dims = (rows, 1100) if len(c["dims"]) == 2 else (rows, 40, 140)
    T = 3 * tile[0] + 5
    a = field(CONFIG_SEEDS[cfg] + 200 + n, dims)
    s = hhc.stencil_create(kind, dims)
    d_in = torch.from_numpy(a).to(DEV)
    d_out = torch.full_like(d_in, float("nan"))
    hhc.stencil_run_dist_local(s, n, d_in, d_out, T, tile, threads, overlap)
    hhc.stencil_destroy(s)
    assert_bits(d_out.cpu().numpy(), oracle.run(kind, a, T, hhc.FUSED), f"{cfg} n={n} tile {tile} x {threads}")
