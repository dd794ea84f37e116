"""CPU-side checks of the C ABI (include/hhc.h / libhhc.so): the library
loads, exports every declared symbol, rejects bad arguments, and its host
parts (planner, model_predict, model_select_tile) agree with the oracle.
No GPU needed (no stencil compute is called here)."""
import math
import random
import re
import os

import pytest

import paper_conf_ppopp_prajapatirradg17_b200 as hhc
from oracle import hex_geometry as hg
from oracle import model_oracle as mo

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def lib():
    from paper_conf_ppopp_prajapatirradg17_b200._build import build
    build()
    return hhc.load()


def header_functions():
    src = open(os.path.join(ROOT, "include", "hhc.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    names = re.findall(r"^\s*(?:const\s+)?[a-z_0-9]+\*?\s+\**([a-z_0-9]+)\s*\(", src, flags=re.M)
    return sorted(set(names))


def test_exports_every_declared_symbol(lib):
    names = header_functions()
    assert len(names) >= 12, names
    for n in names:
        assert hasattr(lib, n), n
    assert set(hhc.EXPORTED_SYMBOLS) == set(names)


def test_strerror(lib):
    assert hhc.strerror(0) == "ok"
    assert "tile" in hhc.strerror(hhc.ETILE)


def test_create_without_gpu_fails_loudly(lib):
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    with pytest.raises(hhc.StencilError) as e:
        hhc.stencil_create(hhc.HEAT2D_9PT, (64, 64))
    assert e.value.status in (hhc.ENODEV, hhc.ECUDA)


def test_tile_validation(lib):
    assert hhc.stencil_tile_resources(2, (8, 8, 64))[1] == 32        # 8 column threads x 4 groups
    for bad in [(7, 8, 64), (0, 8, 64), (8, 0, 64), (8, 8, 48), (8, 8, 0)]:
        with pytest.raises(hhc.StencilError):
            hhc.stencil_tile_resources(2, bad)
    with pytest.raises(hhc.StencilError):
        hhc.stencil_tile_resources(3, (8, 4, 4, 48))
    with pytest.raises(hhc.StencilError):                              # smem > 227 KB
        hhc.stencil_tile_resources(2, (64, 64, 1024))
    with pytest.raises(hhc.StencilError):                              # threads not a multiple
        hhc.stencil_tile_resources(2, (8, 8, 64), threads=20)
    sm, thr, regs = hhc.stencil_tile_resources(3, (8, 4, 4, 32), kind=hhc.HEAT3D_7PT)
    assert regs >= 0                                                  # 0 without a device (unknown)
    assert sm == mo.smem_bytes_exact(3, (8, 4, 4, 32)) and thr == mo.default_threads(3, (8, 4, 4, 32))


def test_plan_info_matches_tiling(lib):
    """Nw and the per-row hexagon counts of the planner vs the brute-force tiling."""
    for tT in (2, 4, 6, 8):
        for tS in (1, 2, 5):
            S1, T = 33, 2 * tT + 3
            rows, w, *_ = hg.analyse(S1, T, tS, tT)
            nrows, wa, wb, _ = hhc.stencil_plan_info((S1 + 2, 40), T, (tT, tS, 32))
            assert nrows == len(rows)
            for m in rows[1:-1]:
                assert w[m] == (wa if m % 2 == 0 else wb)


def hw_pair(kind, geometry, rnd=None, b200=False):
    o = mo.gtx980(kind, geometry)
    if b200:
        o.nSM, o.MSM, o.Mblock = 148, 228 * 1024, 227 * 1024
    if rnd is not None:
        o.L *= rnd.uniform(0.2, 5)
        o.C_iter *= rnd.uniform(0.2, 5)
        o.tau_sync *= rnd.uniform(0.2, 5)
        o.regs_per_thread = rnd.choice([0, 0, 40, 64])
        if geometry == hhc.EXACT_GW:
            o.window_rows = rnd.choice([0.0, 0.3, 1.0, 2.5])
    c = hhc.make_hw(n_sm=o.nSM, n_v=o.nV, mtb_sm=o.MTBSM, r_sm=o.RSM, m_sm_bytes=o.MSM,
                    m_block_bytes=o.Mblock, L_s_per_word=o.L, tau_sync_s=o.tau_sync, T_sync_s=o.T_sync,
                    C_iter_s=o.C_iter, regs_per_thread=o.regs_per_thread, geometry=geometry,
                    window_rows=o.window_rows)
    return o, c


def test_model_predict_matches_oracle_hand_example(lib):
    o, c = hw_pair(3, hhc.PAPER)
    t = hhc.model_predict(hhc.GRADIENT2D, (8194, 8194), 8192, (8, 8, 256), c)
    assert abs(t - mo.talg(2, (8192, 8192), 8192, (8, 8, 256, 0), o)) <= 1e-12 * t
    assert abs(t - 15.96397) < 2e-5


@pytest.mark.parametrize("geometry", [hhc.PAPER, hhc.EXACT, hhc.EXACT_G, hhc.EXACT_GW])
def test_model_predict_matches_oracle_random(lib, geometry):
    rnd = random.Random(geometry + 7)
    n = 0
    for _ in range(400):
        kind = rnd.choice([1, 2, 3, 4, 5, 6])
        nd = hhc.KIND_NDIMS[kind]
        o, c = hw_pair(kind, geometry, rnd, b200=rnd.random() < 0.5)
        if nd == 2:
            S = (rnd.randint(1, 3000), rnd.randint(1, 3000))
            tile = (2 * rnd.randint(1, 20), rnd.randint(1, 40), 32 * rnd.randint(1, 12), 0)
        else:
            S = (rnd.randint(1, 300), rnd.randint(1, 300), rnd.randint(1, 300))
            tile = (2 * rnd.randint(1, 10), rnd.randint(1, 12), rnd.randint(1, 8), 32 * rnd.randint(1, 4))
        T = rnd.randint(1, 500)
        dims = tuple(s + 2 for s in S)
        got = hhc.model_predict(kind, dims, T, tile, c)
        exp = mo.talg(nd, S, T, tile, o)
        if math.isinf(exp):
            assert math.isinf(got)
        else:
            n += 1
            assert abs(got - exp) <= 1e-12 * exp, (kind, S, T, tile, got, exp)
    assert n > 100


@pytest.mark.parametrize("overlap", [0, 1])
def test_model_predict_multi_gpu_matches_oracle(lib, overlap):
    """Reading M7 (the slab model, BASELINE north_star): C++ talg_dist vs the
    oracle's transcription, random problems, G in 2..8, both exchange variants,
    both geometries."""
    rnd = random.Random(70 + overlap)
    n = 0
    for _ in range(200):
        kind = rnd.choice([1, 2, 3, 4, 5])
        nd = hhc.KIND_NDIMS[kind]
        geometry = rnd.choice([hhc.PAPER, hhc.EXACT, hhc.EXACT_G, hhc.EXACT_GW])
        o, c = hw_pair(kind, geometry, rnd, b200=True)
        G = rnd.randint(2, 8)
        o.n_gpus = c.n_gpus = G
        o.link_Bps = c.link_bytes_per_s = rnd.choice([0.0, 7.7e11, 5e10])
        o.link_lat = c.link_latency_s = rnd.choice([0.0, 1e-5])
        o.dist_overlap = c.dist_overlap = overlap
        if nd == 2:
            S = (rnd.randint(50, 3000), rnd.randint(1, 2000))
            tile = (2 * rnd.randint(1, 12), rnd.randint(1, 30), 32 * rnd.randint(1, 8), 0)
        else:
            S = (rnd.randint(30, 300), rnd.randint(1, 200), rnd.randint(1, 200))
            tile = (2 * rnd.randint(1, 6), rnd.randint(1, 10), rnd.randint(1, 8), 32 * rnd.randint(1, 3))
        T = rnd.randint(1, 300)
        got = hhc.model_predict(kind, tuple(s + 2 for s in S), T, tile, c)
        exp = mo.talg(nd, S, T, tile, o)
        if math.isinf(exp):
            assert math.isinf(got)
        else:
            n += 1
            assert abs(got - exp) <= 1e-12 * exp, (kind, S, T, tile, G, got, exp)
    assert n > 50


def test_model_predict_invalid_and_infeasible(lib):
    _, c = hw_pair(2, hhc.PAPER)
    assert math.isnan(hhc.model_predict(hhc.HEAT2D_9PT, (64, 64), 10, (7, 4, 32), c))
    assert math.isnan(hhc.model_predict(hhc.HEAT2D_9PT, (64, 64, 64), 10, (8, 4, 32), c))
    assert math.isnan(hhc.model_predict(hhc.HEAT2D_9PT, (64, 64), 0, (8, 4, 32), c))
    assert math.isinf(hhc.model_predict(hhc.HEAT2D_9PT, (4098, 4098), 64, (16, 64, 1024), c))


@pytest.mark.parametrize("geometry", [hhc.PAPER, hhc.EXACT])
@pytest.mark.parametrize("kind,S,T", [(2, (60, 70), 12), (3, (45, 100), 9), (4, (20, 18, 40), 6),
                                      (1, (130, 33), 5)])
def test_select_tile_matches_oracle(lib, geometry, kind, S, T):
    o, c = hw_pair(kind, geometry, b200=True)
    nd = hhc.KIND_NDIMS[kind]
    best, thr, cands = hhc.model_select_tile(kind, tuple(s + 2 for s in S), T, c, 0.10)
    ob, ot, oc = mo.select_tile(nd, S, T, o, 0.10)
    assert best == ob
    assert cands == oc
    assert thr == mo.default_threads(nd, best)


def test_select_tile_infeasible(lib):
    _, c = hw_pair(2, hhc.PAPER)
    c.m_block_bytes = 16
    with pytest.raises(hhc.StencilError):
        hhc.model_select_tile(hhc.HEAT2D_9PT, (66, 66), 10, c)


def test_exact_fit_recovers_constants(lib):
    """tune.fit_exact (reading Q14, EXACT): compute-only times generated as
    C * A + tau * B are fitted back to (C, tau) (relative least squares)."""
    import random
    from paper_conf_ppopp_prajapatirradg17_b200 import tune
    rnd = random.Random(3)
    C, tau = 1.3e-8, 2.5e-7
    insts = []
    while len(insts) < 25:
        dims = (rnd.randint(1024, 4096), rnd.randint(1024, 4096))
        T = rnd.randint(16, 64)
        tile = tune.random_tile(rnd, 2, dims)
        a = tune._basis(hhc.HEAT2D_9PT, dims, T, tile, 1.0, 0.0)
        b = tune._basis(hhc.HEAT2D_9PT, dims, T, tile, 0.0, 1.0)
        if not (math.isfinite(a) and math.isfinite(b)):
            continue
        insts.append((dims, T, tile, (C * a + tau * b) / a))
    fit = tune.fit_exact(hhc.HEAT2D_9PT, insts)
    assert abs(fit["C_iter_s"] / C - 1) < 1e-6 and abs(fit["tau_level_s"] / tau - 1) < 1e-6
    assert fit["rel_rmse"] < 1e-9


# ---- Jacobi-1D: the paper's 1D model (Section 4.1) and the library agree
@pytest.mark.parametrize("geometry", [hhc.PAPER, hhc.EXACT])
def test_model_1d_matches_oracle(lib, geometry):
    rnd = random.Random(geometry + 70)
    n = 0
    for _ in range(200):
        o, c = hw_pair(1, geometry, rnd, b200=rnd.random() < 0.5)   # C_iter: a parameter (Table 4 has no 1D row)
        S = (rnd.randint(1, 10 ** 6),)
        tile = (2 * rnd.randint(1, 200), rnd.randint(1, 3000), 0, 0)
        T = rnd.randint(1, 2000)
        got = hhc.model_predict(hhc.JACOBI1D_3PT, (S[0] + 2,), T, tile, c)
        exp = mo.talg(1, S, T, tile, o)
        if math.isinf(exp):
            assert math.isinf(got)
        else:
            n += 1
            assert abs(got - exp) <= 1e-12 * exp, (S, T, tile, got, exp)
    assert n > 100
    o, c = hw_pair(1, geometry, b200=True)
    best, thr, cands = hhc.model_select_tile(hhc.JACOBI1D_3PT, (3000,), 40, c, 0.10)
    ob, ot, oc = mo.select_tile(1, (2998,), 40, o, 0.10)
    assert best == ob and cands == oc and thr == 256


def test_model_1d_hand_example():
    """Eqs. 3-9, 10 and 6 by hand for S = 1000, T = 10, tile (4, 8), GTX 980 constants (Jacobi2D C_iter):
    Nw = 2*ceil(10/4) + eps = 6 (r = 10 - 8 = 2 <= tT/2 -> eps = 0); w = ceil(1000/20) = 50;
    mio = 2(8+8) = 32 words; wtile = 10: c = 2 Citer (ceil(8/128) + ceil(10/128)) + 4 tau = 4 Citer + 4 tau;
    Mtile = 2(8+4) = 24 words = 96 B -> k = min(98304 // 96, 32) = 32 -> Ttile = m' + c + 31 max(m', c);
    rounds = ceil(ceil(50/32)/16) = 1."""
    o = mo.gtx980(1, mo.PAPER)
    Nw, w = 6, 50
    m = 32 * o.L + 2 * o.tau_sync
    c = 4 * o.C_iter + 4 * o.tau_sync
    Ttile = m + c + 31 * max(m, c)
    exp = Nw * Ttile * 1 + Nw * o.T_sync
    assert abs(mo.talg(1, (1000,), 10, (4, 8, 0, 0), o) - exp) <= 1e-15 * exp


def test_leff_fit_recovers_L(lib):
    """tune.fit_leff (reading Q14b): full-run times generated by the EXACT model
    with a known per-word cost L* are fitted back to L* (C_iter/tau held)."""
    from paper_conf_ppopp_prajapatirradg17_b200 import tune
    cal = {"L_s_per_word": 6.5e-13, "tau_sync_s": 1.5e-8, "T_sync_s": 5.4e-7, "C_iter_s": {"4": 4e-9},
           "exact_fit": {"4": {"C_iter_s": 4e-9, "tau_level_s": 5e-10}}}
    rnd = random.Random(3)
    Lstar = 2.1e-11
    full = []
    for _ in range(25):
        dims = (rnd.randint(96, 256), rnd.randint(96, 256), rnd.randint(96, 256))
        tile = (2 * rnd.randint(1, 6), rnd.randint(1, 8), rnd.randint(1, 6), 32 * rnd.randint(1, 2))
        T = rnd.randint(8, 24)
        hw = tune.b200_hw(cal, 4, hhc.EXACT)
        hw.L_s_per_word = Lstar
        t = hhc.model_predict(4, dims, T, tile, hw)
        if math.isfinite(t):
            full.append((dims, T, tile, t))
    fit = tune.fit_leff(cal, 4, full)
    assert abs(fit["L_s_per_word"] / Lstar - 1) < 1e-3 and fit["rel_rmse"] < 1e-3 and fit["n"] == len(full)


@pytest.mark.parametrize("geometry", [hhc.EXACT, hhc.EXACT_G, hhc.EXACT_GW])
def test_exact_fit_recovers_planted_constants(lib, geometry):
    """tune.fit_exact (reading Q14; M10 for EXACT_GW): compute-only times generated
    by the model of `geometry` with planted C_iter, tau (and window_rows), recorded
    the way the calibration records them (as C_iter samples v = T / the
    micro-benchmark's own EXACT count), are fitted back to the planted constants."""
    from paper_conf_ppopp_prajapatirradg17_b200 import tune
    kind = hhc.HEAT2D_9PT if geometry != hhc.EXACT_GW else hhc.HEAT3D_7PT
    C, tau, w = 1.3e-8, 2.2e-8, 0.7
    rnd = random.Random(11 + geometry)
    insts = []
    while len(insts) < 40:
        if kind == hhc.HEAT2D_9PT:
            dims = (rnd.randint(1024, 4096), rnd.randint(1024, 4096))
            tile = (2 * rnd.randint(1, 16), rnd.randint(1, 32), 32 * rnd.randint(1, 16), 0)
            T = rnd.randint(16, 64)
        else:
            dims = (rnd.randint(96, 256), rnd.randint(96, 256), rnd.randint(96, 256))
            tile = (2 * rnd.randint(1, 6), rnd.randint(1, 8), rnd.randint(1, 6), 32 * rnd.randint(1, 2))
            T = rnd.randint(8, 24)
        hw = tune.b200_hw(None, kind, geometry)
        hw.C_iter_s, hw.tau_sync_s, hw.L_s_per_word, hw.T_sync_s = C, tau, 0.0, 0.0
        hw.window_rows = w if geometry == hhc.EXACT_GW else 0.0
        t = hhc.model_predict(kind, dims, T, tile, hw)
        cnt = tune._micro_count(kind, dims, T, tile)
        if math.isfinite(t) and math.isfinite(cnt) and cnt > 0:
            insts.append((dims, T, tile, t / cnt))
    fit = tune.fit_exact(kind, insts, geometry)
    # the model is linear in (C_iter, tau, C_iter * window_rows) up to Eq. 16's max(m', c) on
    # time-clipped rows (m' = 2 tau when L = 0): near-exact, not exact
    tol = 1e-2 if kind == hhc.HEAT2D_9PT else 5e-2           # 3D: more rows where m' > c
    assert fit["rel_rmse"] < tol and fit["n"] == len(insts), fit
    assert abs(fit["C_iter_s"] / C - 1) < tol and abs(fit["tau_level_s"] / tau - 1) < 2 * tol, fit
    if geometry == hhc.EXACT_GW:
        assert abs(fit["window_rows"] / w - 1) < 4 * tol, fit


@pytest.mark.parametrize("geometry", [hhc.PAPER, hhc.EXACT])
def test_model_radius_r_matches_oracle(lib, geometry):
    """f4 kinds (radius R = 2..4, reading F4): C++ model_predict vs the oracle,
    random problems and tiles; model_select_tile's argmin and candidates too."""
    rnd = random.Random(90 + geometry)
    n = 0
    for _ in range(150):
        kind = rnd.choice([8, 9, 10])
        R = hhc.KIND_RADIUS[kind]
        o, c = hw_pair(kind if kind < 7 else 1, geometry, rnd, b200=True)
        S = rnd.randint(50, 200000)
        tile = (2 * rnd.randint(1, 64), rnd.randint(1, 3000), 0, 0)
        T = rnd.randint(1, 500)
        got = hhc.model_predict(kind, (S + 2 * R,), T, tile, c)
        exp = mo.talg(1, (S,), T, tile, o, R)
        if math.isinf(exp):
            assert math.isinf(got)
        else:
            n += 1
            assert abs(got - exp) <= 1e-12 * exp, (kind, S, T, tile, got, exp)
    assert n > 50
    o, c = hw_pair(1, geometry, b200=True)
    best, thr, cands = hhc.model_select_tile(9, (5000 + 6,), 64, c, 0.10)
    ob, ot, oc = mo.select_tile(1, (5000,), 64, o, 0.10, R=3)
    assert best == ob and cands == oc
