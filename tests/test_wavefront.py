"""Wavefront-parallel Jacobi-1D (reading W1), CPU side.

PAPER.md L1160-1170: "Consider, wavefront parallel Jacobi1D stencil. The total
execution time is the sum of the times for each wavefront ... equation 6 holds
for wavefront parallel codes."

* The oracle's tile set (oracle.model_oracle.wavefront_tiles) is pinned from
  first principles: every interior point (t, x) lies in exactly one listed
  tile, and each of its three inputs (t-1, x-1..x+1) is produced by the same
  tile or by a tile of an EARLIER wavefront (or is level 0 / the ring) --
  i.e. the launches are a valid schedule of Eq. 1.
* The oracle's Talg is pinned by a hand-computed case.
* The library's schedule (stencil_wavefront_info) and model
  (model_predict_wavefront) agree with the oracle.
"""
import math
import random

import pytest

import paper_conf_ppopp_prajapatirradg17_b200 as hhc
from oracle import model_oracle as mo


@pytest.fixture(scope="module")
def lib():
    from paper_conf_ppopp_prajapatirradg17_b200._build import build
    build()
    return hhc.load()


def brute_owner(S, T, tT, tS):
    """(t, x) -> (i, j) for every interior point, from the tile definition
    (levels (i tT, (i+1) tT], skewed columns [j tS, (j+1) tS))."""
    own = {}
    for t in range(1, T + 1):
        for x in range(1, S + 1):
            own[(t, x)] = ((t - 1) // tT, (x + t) // tS)
    return own


@pytest.mark.parametrize("S,T,tT,tS", [(6, 2, 2, 4), (10, 7, 3, 2), (13, 9, 4, 5), (1, 5, 2, 2),
                                       (20, 1, 1, 3), (17, 16, 5, 7), (9, 30, 8, 3)])
def test_tiles_partition_and_schedule_valid(S, T, tT, tS):
    waves = mo.wavefront_tiles(S, T, tT, tS)
    listed = {}
    for d, tiles in waves.items():
        for (i, j, nlev) in tiles:
            assert i + j == d
            assert nlev == min((i + 1) * tT, T) - i * tT
            listed[(i, j)] = d
    own = brute_owner(S, T, tT, tS)
    # exactly the tiles that own a point are listed
    assert set(own.values()) == set(listed)
    for (t, x), (i, j) in own.items():
        d = listed[(i, j)]
        for xx in (x - 1, x, x + 1):
            if t - 1 == 0 or xx in (0, S + 1):
                continue                      # level 0 or the fixed ring: input data
            src = own[(t - 1, xx)]
            assert src == (i, j) or listed[src] < d, ((t, x), (t - 1, xx), src, (i, j))


def test_talg_wavefront_hand_example():
    """S = 6, T = 2, tile (2, 4): one band, tiles j = 0, 1, 2 (x' in [0, 3], [4, 7], [8, 11]
    each meet x = x' - t in [1, 6] for t in {1, 2}; j = 3 would need x' - 2 <= 6 with x' >= 12),
    so 3 wavefronts of one tile with nlev = 2.  With L = tau = 0, T_sync = 1, C_iter = 1,
    nV = 4, MTBSM = 1 (k = 1): c = 2 ceil(4/4) = 2, Ttile = 2, Talg = 3 (1 + 2) = 9."""
    hw = mo.HW(nSM=1, nV=4, MTBSM=1, RSM=65536, MSM=1 << 20, Mblock=1 << 20, L=0.0,
               tau_sync=0.0, T_sync=1.0, C_iter=1.0)
    assert sorted(mo.wavefront_tiles(6, 2, 2, 4)) == [0, 1, 2]
    assert mo.talg_wavefront_1d(6, 2, (2, 4), hw) == 9.0
    # Eq. 12 with k = 2 tiles per SM: Ttile = m' + c + (k-1) max(m', c) = 4 per wavefront
    hw.MTBSM = 2
    assert mo.talg_wavefront_1d(6, 2, (2, 4), hw) == 3 * (1 + 4)
    # EXACT (reading W2): one tile per wavefront -> the busiest SM holds one tile, Ttile = 2 again
    hw.geometry = mo.EXACT
    assert mo.talg_wavefront_1d(6, 2, (2, 4), hw) == 9.0


def test_library_schedule_matches_oracle(lib):
    rnd = random.Random(3)
    for _ in range(300):
        S = rnd.randint(1, 3000)
        T = rnd.randint(1, 300)
        tT = rnd.randint(1, 40)
        tS = rnd.randint(2, 600)
        waves = mo.wavefront_tiles(S, T, tT, tS)
        nw, nt, mx = hhc.stencil_wavefront_info((S + 2,), T, (tT, tS))
        assert nw == len(waves)
        assert nt == sum(len(v) for v in waves.values())
        assert mx == max(len(v) for v in waves.values())


@pytest.mark.parametrize("geometry", [hhc.PAPER, hhc.EXACT])
def test_library_model_matches_oracle(lib, geometry):
    rnd = random.Random(11 + geometry)
    n = 0
    for _ in range(150):
        o = mo.gtx980(1, geometry)
        if rnd.random() < 0.5:
            o.nSM, o.MSM, o.Mblock = 148, 228 * 1024, 227 * 1024
        o.L *= rnd.uniform(0.2, 5)
        o.C_iter *= rnd.uniform(0.2, 5)
        o.tau_sync *= rnd.uniform(0.2, 5)
        o.regs_per_thread = rnd.choice([0, 0, 40])
        c = hhc.make_hw(n_sm=o.nSM, n_v=o.nV, mtb_sm=o.MTBSM, r_sm=o.RSM, m_sm_bytes=o.MSM,
                        m_block_bytes=o.Mblock, L_s_per_word=o.L, tau_sync_s=o.tau_sync, T_sync_s=o.T_sync,
                        C_iter_s=o.C_iter, regs_per_thread=o.regs_per_thread, geometry=geometry)
        S = rnd.randint(1, 20000)
        T = rnd.randint(1, 200)
        tile = (rnd.randint(1, 64), rnd.randint(2, 16000))
        got = hhc.model_predict_wavefront((S + 2,), T, tile, c)
        exp = mo.talg_wavefront_1d(S, T, tile, o)
        if math.isinf(exp):
            assert math.isinf(got)
        else:
            n += 1
            assert abs(got - exp) <= 1e-12 * exp, (S, T, tile, got, exp)
    assert n > 60
    assert math.isnan(hhc.model_predict_wavefront((2,), 5, (2, 4), c))
    assert math.isnan(hhc.model_predict_wavefront((100,), 5, (2, 1), c))


@pytest.mark.parametrize("geometry", [hhc.PAPER, hhc.EXACT])
def test_library_select_matches_oracle(lib, geometry):
    o = mo.gtx980(1, geometry)
    o.nSM, o.MSM, o.Mblock = 148, 228 * 1024, 227 * 1024
    c = hhc.make_hw(n_sm=o.nSM, n_v=o.nV, mtb_sm=o.MTBSM, r_sm=o.RSM, m_sm_bytes=o.MSM,
                    m_block_bytes=o.Mblock, L_s_per_word=o.L, tau_sync_s=o.tau_sync, T_sync_s=o.T_sync,
                    C_iter_s=o.C_iter, geometry=geometry)
    for S, T in ((500, 24), (61, 9)):
        best, cands = hhc.model_select_wavefront_tile((S + 2,), T, c, 0.10)
        ob, ot, oc = mo.select_tile_wavefront(S, T, o, 0.10)
        assert best == ob and cands == oc
        assert ot == min(mo.talg_wavefront_1d(S, T, tl, o) for tl in oc)
