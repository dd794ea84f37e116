"""oracle/hex_geometry.py -- TEST INFRASTRUCTURE ONLY.

Brute-force enumeration of the hexagonal tiling of the (t, S1) iteration
space (§3.1 and Fig. 1; §4.1): staggered
hexagons of base tS and height tT, pitch 2tS + tT, one "row of hexagons" per
kernel launch.  Points are assigned to tiles by testing membership in every
candidate hexagon (no closed forms), so the counts derived here pin the
closed forms used by model_oracle.py (EXACT geometry) and by the product's
planner, and the dependence check pins the legality of the schedule.

Hexagon shape (reading G1): the tile with bottom-left corner
(t0, x0) holds the points (t0 + tau, x) for tau in [0, tT) and
x0 - m(tau) <= x < x0 + tS + m(tau), with m(tau) = min(tau, tT - tau).
Lattice (reading G2): phase A corners at (1 + k*tT, 1 + j*P), phase B corners
at (1 - tT/2 + k*tT, 1 + tS + tT/2 + j*P); the row index of a tile is
m = (t0 - 1) / (tT/2), even for A, odd for B.

Radius R (reading F4; "the slopes of the
hexagons change by constant factors"): m(tau) = R min(tau, tT - tau), pitch
P = 2tS + R tT, phase B corners at x = 1 + tS + R tT/2 + j*P, and a point
depends on (t-1, x-R .. x+R).  R = 1 is the paper's first-order case.
"""
from __future__ import annotations

from collections import defaultdict


def hexagon_rows(tS: int, tT: int):
    return [(tau, -min(tau, tT - tau), tS + min(tau, tT - tau)) for tau in range(tT)]


def tile_of(t: int, x: int, tS: int, tT: int, R: int = 1):
    """Return the unique (m, j) whose hexagon contains (t, x); raises if the
    point is covered zero or several times."""
    P = 2 * tS + R * tT
    h = tT // 2
    hits = []
    # candidate rows: the point's level lies in [t0, t0 + tT)
    for m in range((t - 1) // h - 2, (t - 1) // h + 2):
        t0 = 1 + m * h
        tau = t - t0
        if not (0 <= tau < tT):
            continue
        base = 1 if m % 2 == 0 else 1 + tS + R * h
        mm = R * min(tau, tT - tau)
        # x0 - mm <= x < x0 + tS + mm with x0 = base + j*P
        for j in range((x - base - tS - mm) // P - 1, (x - base + mm) // P + 2):
            x0 = base + j * P
            if x0 - mm <= x < x0 + tS + mm:
                hits.append((m, j))
    if len(hits) != 1:
        raise AssertionError(f"point {(t, x)} covered {len(hits)} times: {hits}")
    return hits[0]


def enumerate_tiling(S1: int, T: int, tS: int, tT: int, R: int = 1):
    """Map every point of [1,T] x [1,S1] to its tile.  Returns
    tiles: {(m, j): set of (t, x)}."""
    tiles = defaultdict(set)
    for t in range(1, T + 1):
        for x in range(1, S1 + 1):
            tiles[tile_of(t, x, tS, tT, R)].add((t, x))
    return tiles


def analyse(S1: int, T: int, tS: int, tT: int, R: int = 1):
    """Brute-force statistics of the tiling:
    rows: sorted list of non-empty row indices (= kernel launches, Nw);
    w: {m: number of non-empty tiles in row m};
    reads/writes: {(m, j): number of global reads (values the tile needs that
    it does not compute, excluding the fixed ring x = 0, S1+1) and facet
    writes (values it computes that some other tile reads, or at t = T)};
    and checks the schedule: every dependence (t-1, x+d) of a point is either
    level 0 / the ring, in the same tile at an earlier level, or in a tile of
    an EARLIER row (never the same row)."""
    tiles = enumerate_tiling(S1, T, tS, tT, R)
    owner = {}
    for key, pts in tiles.items():
        for p in pts:
            owner[p] = key
    rows = sorted({k[0] for k in tiles})
    w = defaultdict(int)
    for (m, j) in tiles:
        w[m] += 1
    reads = defaultdict(int)
    writes = defaultdict(int)
    for key, pts in tiles.items():
        need = set()
        for (t, x) in pts:
            for d in range(-R, R + 1):
                q = (t - 1, x + d)
                if q[0] == 0 or q[1] < 1 or q[1] > S1:
                    continue            # initial value or ring: read from the input
                ok = owner[q]
                if ok == key:
                    continue
                if ok[0] >= key[0]:
                    raise AssertionError(f"dependence {q}->{(t, x)} not from an earlier row")
                need.add(q)
        reads[key] = len(need)
        wr = 0
        for (t, x) in pts:
            if t == T:
                wr += 1
                continue
            for d in range(-R, R + 1):
                q = (t + 1, x + d)
                if 1 <= q[1] <= S1 and owner[q] != key:
                    wr += 1
                    break
        writes[key] = wr
    return rows, dict(w), dict(reads), dict(writes), tiles
