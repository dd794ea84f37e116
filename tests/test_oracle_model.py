"""Pins of the model oracle (oracle/model_oracle.py) and of the hexagon
geometry readings, against hand arithmetic from the paper's own constants,
the paper's special cases, a brute-force enumeration of the tiling, and
invariants.  PAPER.md §4 (Eqs. 2-30), §5 Tables 2-4, §6.1 (Eq. 31)."""
import math
import random

import pytest

from oracle import hex_geometry as hg
from oracle import model_oracle as mo


def test_hand_worked_gradient2d_gtx980():
    """Re-derived by hand from Tables 2-4 for the Fig. 5 problem
    (Gradient-2D, S1 = S2 = T = 8192) at tile
    (tT, tS1, tS2) = (8, 8, 256), literal equations:
      Nw = 2*1024 + 1 = 2049          (Eq. 3, T mod tT = 0 -> eps = 1)
      wtile = 14                       (Eq. 4)
      w = ceil(8192/24) = 342          (Eq. 5)
      Mtile = 2*17*265 = 9010 words = 36040 B <= 48 KB      (Eq. 19)
      k = min(32, floor(98304/36040)) = 2                   (Eq. 11/31)
      mi = mo = 256*(8+16) = 6144      (Eq. 13)
      L = 7.36e-3 s/GB * 4e-9 = 2.944e-11 s/word
      m' = 12288*2.944e-11 + 2*7.96e-10 = 3.63355e-7 s       (Eq. 14)
      c = 2*6.09e-8*(16+20+24+28) + 8*7.96e-10 = 1.0724768e-5 s  (Eq. 15)
      N2 = ceil(8200/256) = 33
      Tprism = m' + 2*c*33 = 7.0819804e-4 s                (Eq. 16, k > 1)
      rounds = ceil(ceil(342/2)/16) = 11
      Talg = 2049*9.24e-7 + 2049*7.0819804e-4*11 = 15.96397 s   (Eq. 17)"""
    hw = mo.gtx980(3)
    assert mo.Nw_eq3(8192, 8) == 2049
    assert mo.wtile_eq4(8, 8) == 14
    assert mo.w_eq5(8192, 8, 8) == 342
    assert abs(mo.c_eq15(8, 8, 256, hw) - 1.0724768e-5) < 1e-15
    t = mo.talg(2, (8192, 8192), 8192, (8, 8, 256, 0), hw)
    assert abs(t - 15.96397) < 2e-5, t


def test_Nw_eq3_equals_exact_row_count():
    """Eq. 3 with its eps rule is exactly ceil(2T/tT)+1 (reading G2), and both
    equal the number of non-empty hexagon rows of a brute-force tiling."""
    for tT in range(2, 34, 2):
        for T in range(1, 200):
            assert mo.Nw_eq3(T, tT) == math.ceil(2 * T / tT) + 1
    for tT in (2, 4, 6, 8):
        for tS in (1, 2, 3, 5):
            for T in (1, 2, 5, 8, 13):
                rows, *_ = hg.analyse(25, T, tS, tT)
                assert len(rows) == mo.Nw_eq3(T, tT), (tT, tS, T)
                assert rows == list(range(-1, len(rows) - 1))
                assert len(list(mo.rows_exact(T, tT))) == len(rows)


def test_tiling_is_a_legal_schedule_and_w_counts():
    """Exact cover (tile_of raises otherwise), dependences only on earlier rows,
    and the per-row hexagon counts of reading G2."""
    for tT in (2, 4, 6, 8):
        for tS in (1, 2, 4, 7):
            S1, T = 37, 3 * tT + 1
            rows, w, _, _, _ = hg.analyse(S1, T, tS, tT)
            wA, wB = mo.w_rows_exact(S1, tS, tT)
            for m in rows[1:-1]:               # full-height rows
                assert w[m] == (wA if m % 2 == 0 else wB), (tT, tS, m)


def test_exact_footprints_match_enumeration():
    """Reading G3: an interior hexagon reads tS1+2tT+2 values it did not
    compute and writes tS1+2tT-2 facets (per unit inner extent)."""
    for tT in (2, 4, 6, 8, 10):
        for tS in (1, 2, 3, 6):
            S1, T = 80, 4 * tT + 3
            rows, w, reads, writes, tiles = hg.analyse(S1, T, tS, tT)
            P = 2 * tS + tT
            for (m, j), pts in tiles.items():
                ts = {t for t, _ in pts}
                xs = {x for _, x in pts}
                if len(pts) != tT * (tS + tT // 2):
                    continue                    # clipped by time or by the ring
                if min(xs) < 3 or max(xs) > S1 - 2 or min(ts) < 2 or max(ts) >= T:
                    continue
                t0 = min(ts)
                r, wr = mo.row_io_exact(tS, tT, 0, tT, t0, T)
                assert reads[(m, j)] == r == tS + 2 * tT + 2, (tT, tS, m, j)
                assert writes[(m, j)] == wr == tS + 2 * tT - 2, (tT, tS, m, j)
            assert P == 2 * tS + tT


def test_hexagon_area():
    """Area of the implemented hexagon = tT*(tS1 + tT/2) (reading G1); the
    paper's wtile = tS+tT-2 row sum (Eq. 9) is tT*(tS1 + tT/2 - 1)."""
    for tT in range(2, 40, 2):
        for tS in range(1, 30):
            assert sum(mo.row_width(t, tS, tT) for t in range(tT)) == tT * (tS + tT // 2)
            paper = 2 * sum(range(tS, mo.wtile_eq4(tS, tT) + 1, 2))
            assert paper == tT * (tS + tT // 2 - 1)


def test_special_case_wide_vector_units():
    """if nV >= wtile*tS2 every row takes one Citer, so
    c = tT*(Citer + tau_sync)."""
    hw = mo.gtx980(1)
    hw.nV = 10 ** 9
    for tT, tS1, tS2 in [(2, 1, 32), (8, 8, 64), (16, 5, 128)]:
        assert math.isclose(mo.c_eq15(tS1, tT, tS2, hw), tT * (hw.C_iter + hw.tau_sync), rel_tol=1e-12)


def test_k_equals_1_hand_example():
    """Eq. 16's k = 1 branch (Tprism = (m' + c) * N2), worked by hand on a
    B200-sized shared memory (MSM = 228 KB, Mblock = 227 KB) with round
    constants L = 1e-12 s/word, tau_sync = 1e-9 s, T_sync = 2e-6 s,
    Citer = 1e-8 s; Heat-2D, S1 = S2 = 8192, T = 1024, tile (16, 20, 512):
      Nw = 2*64 + 1 = 129                (Eq. 3, T mod tT = 0 -> eps = 1)
      w = ceil(8192 / 56) = 147          (Eq. 5)
      Mtile = 2*37*529 = 39146 words = 156584 B  (Eq. 19)
      k = min(floor(233472 / 156584), 32) = 1    (Eq. 11)
      mi = mo = 512*(20+32) = 26624      (Eq. 13)
      m' = 53248e-12 + 2e-9 = 5.5248e-8 s        (Eq. 14)
      c = 2e-8 * sum_{x=20,22..34} ceil(512x/128) + 16e-9
        = 2e-8 * 4*216 + 1.6e-8 = 1.7296e-5 s   (Eq. 15)
      N2 = ceil(8208/512) = 17
      Tprism = (m' + c) * N2 = 1.7351248e-5 * 17 = 2.94971216e-4 s  (Eq. 16, k = 1)
      rounds = ceil(ceil(147/1)/148) = 1
      Talg = 129*2e-6 + 129*2.94971216e-4*1 = 0.038309286864 s  (Eq. 17)"""
    hw = mo.HW(nSM=148, nV=128, MTBSM=32, RSM=65536, MSM=228 * 1024, Mblock=227 * 1024, L=1e-12,
               tau_sync=1e-9, T_sync=2e-6, C_iter=1e-8)
    assert mo.Nw_eq3(1024, 16) == 129
    assert mo.w_eq5(8192, 20, 16) == 147
    assert math.isclose(mo.c_eq15(20, 16, 512, hw), 1.7296e-5, rel_tol=1e-12)
    t = mo.talg(2, (8192, 8192), 1024, (16, 20, 512, 0), hw)
    assert math.isclose(t, 0.038309286864, rel_tol=1e-11), t
    # one more MTBSM-limited block per SM would be k = 2: the k > 1 branch differs
    hw.MSM = 2 * 156584
    assert not math.isclose(mo.talg(2, (8192, 8192), 1024, (16, 20, 512, 0), hw), 0.038309286864, rel_tol=1e-6)


def test_hand_worked_heat3d_gtx980_paper():
    """The PAPER-literal 3D model (Eqs. 20-30) worked by
    hand on the GTX 980 constants (Tables 2-4: nSM = 16, nV = 128, MTBSM = 32,
    MSM = 96 KB, Mblock = 48 KB, L = 7.36e-3 s/GB -> 2.944e-11 s/word,
    tau_sync = 7.96e-10 s, T_sync = 9.24e-7 s, Citer(Heat3D) = 1.55e-7 s) for
    Heat-3D, S1 = S2 = S3 = 384 (a size of P:L1179-1195), T = 128, tile
    (tT, tS1, tS2, tS3) = (4, 4, 4, 32):
      Nw = 2*32 + 1 = 65                  (Eq. 20 with Eq. 3's eps, T mod tT = 0)
      w = ceil(384 / 12) = 32             (Eq. 22, pitch 2tS1 + tT, reading M2)
      mi = mo = 4*32*(4+8) = 1536 words   (Eq. 24)
      m' = 3072*2.944e-11 + 2*7.96e-10 = 9.203168e-8 s            (Eq. 25)
      wtile = 4 + 4 - 2 = 6;  x = 4, 6:  ceil(4*128/128) + ceil(6*128/128) = 10
      c = 2*1.55e-7*10 + 4*7.96e-10 = 3.103184e-6 s               (Eq. 27)
      Mtile = 2*9*9*37 = 5994 words = 23976 B <= 48 KB            (reading M3)
      k = min(floor(98304/23976), 32) = 4                          (Eq. 11)
      Nsslabs = ceil((388/4)*(388/32)) = ceil(97*12.125) = 1177   (Eq. 23 as printed)
      zeta = max(m', c) = c
      Tslab = m' + k*zeta*Nsslabs = 9.203168e-8 + 4*3.103184e-6*1177
            = 0.01460988230368 s                                   (Eq. 29)
      rounds = ceil(ceil(32/4)/16) = 1
      Talg = 65*9.24e-7 + 65*0.01460988230368*1 = 0.9497024097392 s  (Eq. 30)"""
    hw = mo.gtx980(4)
    assert mo.Nw_eq3(128, 4) == 65
    assert mo.w_eq5(384, 4, 4) == 32
    assert math.isclose(mo.c_eq15(4, 4, 4 * 32, hw), 3.103184e-6, rel_tol=1e-12)
    t = mo.talg(3, (384, 384, 384), 128, (4, 4, 4, 32), hw)
    assert math.isclose(t, 0.9497024097392, rel_tol=1e-11), t


def test_multi_gpu_model_hand_example():
    """Reading M7 (not in the paper) worked by hand with a stub single-GPU time:
    PAPER geometry on the k = 1 hardware above is replaced by the closed form
    of a constant per-row cost, so only M7's own arithmetic is checked.
    G = 4, S1 = 1000 -> own = 250, e = 2, g = tT = 8, T = 20 -> tiles 8, 8, 4;
    inner S2 = 100 -> T_exch = 8*100*4 B / 1e9 B/s + 1e-6 = 4.2e-6 s."""
    calls = []

    def fake(nd, S, T, tile, hw, R=1, planes=False):
        calls.append((S[0], T))
        return 1e-6 * S[0] * T                       # 1 us per row-step

    orig = mo.talg_single
    mo.talg_single = fake
    try:
        hw = mo.gtx980(2)
        hw.n_gpus, hw.link_Bps, hw.link_lat = 4, 1e9, 1e-6
        # plain: (266*8 + 266*8 + 266*4) us + 3 * 4.2 us
        t = mo.talg(2, (1000, 100), 20, (8, 8, 64, 0), hw)
        assert math.isclose(t, 1e-6 * 266 * 20 + 3 * 4.2e-6, rel_tol=1e-12), t
        # overlap: interior 250 rows, 2 edge sub-slabs of 24 rows, exchange hidden (250*Tt us >> 4.2 us)
        hw.dist_overlap = 1
        t = mo.talg(2, (1000, 100), 20, (8, 8, 64, 0), hw)
        assert math.isclose(t, 1e-6 * (250 + 2 * 24) * 20, rel_tol=1e-12), t
        # G = 2: one neighbour
        hw.n_gpus, hw.dist_overlap = 2, 0
        t = mo.talg(2, (1000, 100), 20, (8, 8, 64, 0), hw)
        assert math.isclose(t, 1e-6 * 508 * 20 + 3 * 4.2e-6, rel_tol=1e-12), t
    finally:
        mo.talg_single = orig


def test_infeasible_and_invalid_tiles():
    hw = mo.gtx980(2)
    assert math.isinf(mo.talg(2, (4096, 4096), 64, (16, 64, 1024, 0), hw))   # Mtile > 48 KB
    assert math.isnan(mo.talg(2, (4096, 4096), 64, (7, 4, 64, 0), hw))       # tT odd
    assert math.isnan(mo.talg(2, (4096, 4096), 64, (8, 4, 48, 0), hw))       # tS2 not x32
    assert math.isnan(mo.talg(3, (64, 64, 64), 64, (8, 4, 4, 48), hw))       # tS3 not x32


def ideal_compute_bound(S, T, hw):
    return math.prod(S) * T * hw.C_iter / (hw.nSM * hw.nV)


def test_exact_never_beats_ideal_compute_bound():
    """Every update costs Citer per vector unit: EXACT Talg >= prod(S)*T*Citer/(nSM*nV)."""
    rnd = random.Random(1)
    for _ in range(300):
        kind = rnd.choice([1, 2, 3])
        hw = mo.gtx980(kind, mo.EXACT)
        hw.Mblock = 227 * 1024
        hw.MSM = 228 * 1024
        S = (rnd.randint(40, 3000), rnd.randint(40, 3000))
        T = rnd.randint(1, 300)
        tile = (2 * rnd.randint(1, 16), rnd.randint(1, 30), 32 * rnd.randint(1, 8), 0)
        t = mo.talg(2, S, T, tile, hw)
        if math.isfinite(t):
            assert t >= ideal_compute_bound(S, T, hw) * (1 - 1e-12), (S, T, tile)


def test_paper_literal_minimum_is_degenerate():
    """SURVEY/DESIGN reading M1: at the degenerate tile (2, 1, 640) the literal
    equations predict less than the ideal compute bound for the Fig. 5 problem,
    the EXACT geometry does not -- the reason both modes exist."""
    hw = mo.gtx980(3)
    S, T = (8192, 8192), 8192
    ideal = ideal_compute_bound(S, T, hw)
    assert mo.talg(2, S, T, (2, 1, 640, 0), hw) < ideal
    hwx = mo.gtx980(3, mo.EXACT)
    hwx.Mblock, hwx.MSM = 48 * 1024, 96 * 1024
    assert mo.talg(2, S, T, (2, 1, 640, 0), hwx) >= ideal


def test_talg_monotone_in_T():
    for geom in (mo.PAPER, mo.EXACT):
        hw = mo.gtx980(2, geom)
        prev = 0.0
        for T in range(1, 200, 3):
            t = mo.talg(2, (1000, 900), T, (8, 6, 64, 0), hw)
            assert t >= prev
            prev = t


def test_select_tile_small_space():
    """§6.1: the selector is the exhaustive argmin over Eq. 31's space."""
    hw = mo.gtx980(2)
    S, T = (200, 150), 40
    best, tmin, cands = mo.select_tile(2, S, T, hw, tT_max=16, tS1_max=12, inner_max=256)
    allv = [(mo.talg(2, S, T, tl, hw), tl) for tl in mo.enumerate_space(2, S, T, hw, tT_max=16,
                                                                          tS1_max=12, inner_max=256)]
    allv = [(t, tl) for t, tl in allv if math.isfinite(t)]
    assert min(allv)[1] == best and min(allv)[0] == tmin
    assert set(cands) == {tl for t, tl in allv if t <= 1.1 * tmin}
    assert best in cands


def test_xgroup_rows_reading_m9():
    """Reading M9 (EXACT_G): with G x-groups a level costs G*ceil(W/G) rows, so
    EXACT_G >= EXACT, equal when every row width is a multiple of G (G = 1 or
    W(tau) divisible), and larger for some tile whose rows do not split evenly."""
    hw = mo.gtx980(2, mo.EXACT)
    hw.Mblock, hw.MSM = 227 * 1024, 228 * 1024
    hwg = mo.gtx980(2, mo.EXACT_G)
    hwg.Mblock, hwg.MSM = 227 * 1024, 228 * 1024
    S, T = (2000, 1500), 64
    larger = 0
    for tile, thr in [((8, 4, 64, 0), 32), ((8, 4, 64, 0), 8), ((16, 6, 128, 0), 64), ((4, 2, 32, 0), 12)]:
        hw.threads = hwg.threads = thr
        te, tg = mo.talg(2, S, T, tile, hw), mo.talg(2, S, T, tile, hwg)
        G = thr // (tile[2] // 8)
        widths = {mo.row_width(t, tile[1], tile[0]) for t in range(tile[0])}
        if G == 1 or all(w % G == 0 for w in widths):
            assert te == tg
        else:
            assert tg >= te
            larger += tg > te
    assert larger >= 1


# ---- radius R (reading F4)
def test_radius_r_tiling_geometry():
    """Brute force with radius R: exact cover, every dependence (t-1, x-R..x+R)
    from the same tile or an earlier row, per-row hexagon counts and the
    interior footprints tS1 + 2R tT + 2R (reads) / tS1 + 2R tT - 2R (facets)."""
    for R in (2, 3):
        for tT in (2, 4, 6):
            for tS in (1, 3, 5):
                S1, T = 90, 3 * tT + 1
                rows, w, reads, writes, tiles = hg.analyse(S1, T, tS, tT, R)
                wA, wB = mo.w_rows_exact(S1, tS, tT, R)
                for m in rows[1:-1]:
                    assert w[m] == (wA if m % 2 == 0 else wB), (R, tT, tS, m)
                for (m, j), pts in tiles.items():
                    ts = {t for t, _ in pts}
                    xs = {x for _, x in pts}
                    if len(pts) != sum(mo.row_width(t, tS, tT, R) for t in range(tT)):
                        continue
                    if min(xs) < 2 * R + 1 or max(xs) > S1 - 2 * R or min(ts) < 2 or max(ts) >= T:
                        continue
                    r, wr = mo.row_io_exact(tS, tT, 0, tT, min(ts), T, R)
                    assert reads[(m, j)] == r == tS + 2 * R * tT + 2 * R, (R, tT, tS)
                    assert writes[(m, j)] == wr == tS + 2 * R * tT - 2 * R, (R, tT, tS)


def test_radius_r_paper_model_hand_example():
    """Section 4.1's 1D model with reading F4 at R = 2 on the GTX 980 constants
    (Citer of Jacobi2D as a stand-in), S = 4096, T = 64, tile (tT, tS) = (8, 64):
      Nw = 2*8 + 1 = 17                           (Eq. 3, T mod tT = 0)
      wtile = 64 + 2*(8-2) = 76                   (Eq. 4, slope 2)
      w = ceil(4096 / (128 + 16)) = 29            (Eq. 5, pitch 2 tS + R tT)
      m' = 2*(64 + 32)*2.944e-11 + 2*7.96e-10 = 7.24448e-9 s      (Eqs. 7-8)
      c = 2*3.39e-8*(1+1+1+1) + 8*7.96e-10 = 2.77568e-7 s         (Eq. 9, x = 64, 68, 72, 76)
      Mtile = 2*(76 + 4) = 160 words = 640 B -> k = min(98304/640, 32) = 32   (Eq. 11)
      Ttile = m' + c + 31*max(m', c) = 7.24448e-9 + 32*2.77568e-7 = 8.88942048e-6 s  (Eq. 12)
      rounds = ceil(ceil(29/32)/16) = 1
      Talg = 17*8.88942048e-6 + 17*9.24e-7 = 1.6682814816e-4 s    (Eq. 6)"""
    hw = mo.gtx980(1)
    t = mo.talg(1, (4096,), 64, (8, 64, 0, 0), hw, R=2)
    mp = 2 * (64 + 32) * hw.L + 2 * hw.tau_sync
    c = 2 * hw.C_iter * 4 + 8 * hw.tau_sync
    assert math.isclose(mp, 7.24448e-9, rel_tol=1e-12) and math.isclose(c, 2.77568e-7, rel_tol=1e-12)
    assert math.isclose(t, 1.6682814816e-4, rel_tol=1e-11), t
    # R = 1 is the printed model
    assert mo.talg(1, (4096,), 64, (8, 64, 0, 0), hw, R=1) == mo.talg(1, (4096,), 64, (8, 64, 0, 0), hw)


def test_m10_window_rows_term():
    """Reading M10 (EXACT_GW): the x-groups' window-prologue rows.  With
    window_rows = 0 it is EXACT_G (reading M9); with L = tau = T_sync = 0 and
    k = 1 Talg is affine in window_rows (equal steps), and by hand the slope of a
    one-hexagon-row problem is C_iter * G * inner / nV per level per sub-tile:
    Heat-2D S = (20, 512), T = 4, tile (4, 2, 256) with 64 threads (G = 2)."""
    from dataclasses import replace
    hw = mo.gtx980(2, mo.EXACT_G)
    hw.nSM, hw.MSM, hw.Mblock = 148, 228 * 1024, 227 * 1024
    hw.L = hw.tau_sync = hw.T_sync = 0.0
    hw.threads = 64
    S, T, tile = (20, 512), 4, (4, 2, 256, 0)
    g0 = mo.talg(2, S, T, tile, hw)
    gw = [mo.talg(2, S, T, tile, replace(hw, geometry=mo.EXACT_GW, window_rows=w)) for w in (0.0, 1.0, 2.0)]
    assert gw[0] == g0
    assert abs((gw[2] - gw[1]) - (gw[1] - gw[0])) <= 1e-12 * gw[2]
    # by hand: row m has nlev levels and Nsub = ceil((S2 + nlev - 1) / tS2) sub-tiles per
    # prism, run k at a time in ceil(ceil(w / k) / nSM) rounds (Eq. 2, 16 with m' = 0):
    # slope = C_iter * G * tS2 / nV * sum_m nlev_m * Nsub_m * k * rounds_m
    G, nV = 64 // (256 // 8), hw.nV
    assert G == 2
    slope_hand = 0.0
    for m, lo, hi, t0 in mo.rows_exact(T, tile[0]):
        nlev = hi - lo
        w = mo.w_rows_exact(S[0], tile[1], tile[0])[0 if m % 2 == 0 else 1]
        if nlev <= 0 or w == 0:
            continue
        nsub = mo.ceil_div(S[1] + nlev - 1, tile[2])
        k = mo.k_exact(mo.smem_bytes_exact(2, tile), 64, hw)
        rounds = mo.ceil_div(mo.ceil_div(w, k), hw.nSM)
        per = nlev * nsub * rounds * (k if k > 1 else 1)
        slope_hand += hw.C_iter * G * tile[2] / nV * per
    assert abs((gw[1] - gw[0]) - slope_hand) <= 1e-9 * slope_hand, (gw[1] - gw[0], slope_hand)
