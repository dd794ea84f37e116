"""CPU schedule simulator of the product's 2D HHC kernel (hex2d_kernel in
paper_conf_ppopp_prajapatirradg17_b200/csrc/hhc_kernels.cu), mirrored step by
step: launch rows, blocks, sub-tiles, footprint loads, per-level phases with
face save / halo copy, the x-groups of threads, facet writes.  Global planes
carry a LEVEL TAG per cell so every footprint read can be checked to see the
time level it needs (SURVEY §4 "schedule simulator"): a stale or never-written
value raises immediately.  Arithmetic is a tagged average so values are also
checked against a naive reference.  Test infrastructure only."""
from __future__ import annotations

import numpy as np


def cdiv(a, b):
    return -(-a // b)


def plan_rows(dims, T, tile):
    tT, tS1, tS2 = tile[:3]
    S1i = dims[0] - 2
    h = tT // 2
    P = 2 * tS1 + tT
    Nw = cdiv(2 * T, tT) + 1
    wA = cdiv(S1i + h, P)
    wB = cdiv(S1i - tS1, P) if S1i > tS1 else 0
    rows = []
    for m in range(-1, Nw - 1):
        t0 = 1 + m * h
        lo = max(0, 1 - t0)
        hi = min(tT, T - t0 + 1)
        A = m % 2 == 0
        xbase = 1 if A else 1 + tS1 + h
        w = wA if A else wB
        nlev = hi - lo
        n2 = cdiv(dims[1] - 2 + nlev - 1, tS2)
        if nlev > 0 and w > 0:
            rows.append(dict(m=m, t0=t0, lo=lo, hi=hi, xbase=xbase, w=w, n2=n2))
    return rows


class Sim:
    def __init__(self, a, T, tile, G=1):
        self.S1, self.S2 = a.shape
        self.T = T
        self.tT, self.tS1, self.tS2 = tile[:3]
        self.G = G
        self.a = a
        # global planes: value + level tag (-1 = never written)
        self.val = [a.astype(np.float64).copy(), np.full(a.shape, np.nan)]
        self.lvl = [np.zeros(a.shape, int), np.full(a.shape, -1)]
        ring = np.zeros(a.shape, bool)
        ring[0, :] = ring[-1, :] = ring[:, 0] = ring[:, -1] = True
        self.ring = ring
        self.val[1][ring] = a[ring]
        self.lvl[1][ring] = -2          # ring: valid at every level
        self.lvl[0][ring] = -2

    def gread(self, t, x, y):
        p = t & 1
        tag = self.lvl[p][x, y]
        if tag != -2 and tag != t:
            raise AssertionError(f"read level {t} at ({x},{y}) found level {tag}")
        return self.val[p][x, y]

    def gwrite(self, t, x, y, v):
        p = t & 1
        self.val[p][x, y] = v
        self.lvl[p][x, y] = t

    @staticmethod
    def f(R, k):
        # a simple linear stencil (heat 9pt weights) evaluated in float64
        w = [[1 / 16, 1 / 8, 1 / 16], [1 / 8, 1 / 4, 1 / 8], [1 / 16, 1 / 8, 1 / 16]]
        s = 0.0
        for d1 in range(3):
            for d2 in range(3):
                s += w[d1][d2] * R[d1][k + d2]
        return s

    def run(self):
        for r in plan_rows((self.S1, self.S2), self.T, (self.tT, self.tS1, self.tS2)):
            for b in range(r["w"]):
                self.block(r, b)
        return self.val[self.T & 1]

    def hex_row(self, x0, r, lev):
        nlev = r["hi"] - r["lo"]
        if lev < 0 or lev >= nlev:
            return 0, 0
        tau = r["lo"] + lev
        mm = min(tau, self.tT - tau)
        l = max(x0 - mm, 1)
        rr = min(x0 + self.tS1 + mm, self.S1 - 1)
        if rr < l:
            rr = l
        return l, rr

    def footprint(self, x0, r, lev):
        rl, rr = self.hex_row(x0, r, lev)
        pl, pr = self.hex_row(x0, r, lev - 1)
        empty = rl >= rr
        A0, A1 = rl - 1, rr + 1
        first = lev == 0 or pl >= pr
        if first:
            return dict(A0=A0, A1=A1, f1a=A0, f1b=A1, f2a=A1, f2b=A1, ia=A1, ib=A1, first=True, empty=empty)
        f1a, f1b = A0, max(A0, min(A1, pl))
        f2a, f2b = min(A1, max(pr, A0)), A1
        if f2a < f1b:
            f2a = f1b
        ia, ib = max(A0, pl), min(A1, pr)
        if ib < ia:
            ib = ia
        return dict(A0=A0, A1=A1, f1a=f1a, f1b=f1b, f2a=f2a, f2b=f2b, ia=ia, ib=ib, first=False, empty=empty)

    def is_facet(self, x, nl, nr, final):
        if final or nl >= nr:
            return True
        lo, hi = max(x - 1, 1), min(x + 1, self.S1 - 2)
        return not (lo >= nl and hi < nr)

    def block(self, r, b):
        tT, tS1, tS2 = self.tT, self.tS1, self.tS2
        NX = tS1 + tT + 2
        RS = tS2 + 4
        pl = [np.full((NX, RS), np.nan), np.full((NX, RS), np.nan)]
        plt = [np.full((NX, RS), -99), np.full((NX, RS), -99)]      # level tags in smem (absolute)
        face = np.full((2, tT, NX, 2), np.nan)
        facet = np.full((2, tT, NX, 2), -99)
        x0 = r["xbase"] + b * (2 * tS1 + tT)
        xs = x0 - tT // 2 - 1
        nlev = r["hi"] - r["lo"]
        tb = r["t0"] + r["lo"]
        W = tS2 + 2
        ncol = tS2 // 4
        for j2 in range(r["n2"]):
            a = 1 + j2 * tS2
            fc, fn = j2 & 1, (j2 + 1) & 1
            for lev in range(nlev):
                f = self.footprint(x0, r, lev)
                if f["empty"]:
                    continue
                halo_all = f["first"] or j2 == 0
                items = []
                for x in range(f["f1a"], f["f1b"]):
                    items += [(x, c) for c in range(W)]
                for x in range(f["f2a"], f["f2b"]):
                    items += [(x, c) for c in range(W)]
                if halo_all:
                    for x in range(f["ia"], f["ib"]):
                        items += [(x, c) for c in range(2)]
                dpl = 0 if (lev & 1) else 1
                t_src = tb + lev - 1
                for x, c in items:
                    if lev > 0 and (x == 0 or x == self.S1 - 1):
                        continue                  # ring rows: filled per level in the phase
                    y = a - 1 + c - lev
                    v, tag = 0.0, -99
                    if 0 <= y < self.S2:
                        inner = 1 <= y <= self.S2 - 2 and 1 <= x <= self.S1 - 2
                        if inner or True:
                            v = self.gread(t_src, x, y)
                            tag = t_src
                    pp = x - xs
                    if c >= 2 or lev == 0:
                        pl[dpl][pp, c + 2] = v
                        plt[dpl][pp, c + 2] = tag
                    else:
                        face[fc, lev, pp, c] = v
                        facet[fc, lev, pp, c] = tag
            for lev in range(nlev):
                prev, cur = (0, 1) if (lev & 1) else (1, 0)
                for pp in range(NX):
                    for c in range(2):
                        if lev >= 1:
                            face[fn, lev, pp, c] = pl[prev][pp, tS2 + 2 + c]
                            facet[fn, lev, pp, c] = plt[prev][pp, tS2 + 2 + c]
                        xr = xs + pp
                        if lev + 1 < nlev and xr != 0 and xr != self.S1 - 1:
                            pl[cur][pp, 2 + c] = face[fc, lev + 1, pp, c]
                            plt[cur][pp, 2 + c] = facet[fc, lev + 1, pp, c]
                # ring rows of level lev in skewed coordinates (slots 2 .. tS2+3)
                for xr in (0, self.S1 - 1):
                    pp = xr - xs
                    if 0 <= pp < NX:
                        for slot in range(2, tS2 + 4):
                            y = a + slot - 4 - lev
                            pl[cur][pp, slot] = self.a[xr, y] if 0 <= y < self.S2 else 0.0
                            plt[cur][pp, slot] = -2
                rl, rr = self.hex_row(x0, r, lev)
                nl, nr = self.hex_row(x0, r, lev + 1)
                if rl >= rr:
                    continue
                new = []
                L = rr - rl
                seg = cdiv(L, self.G)
                for grp in range(self.G):
                    xa, xe = rl + grp * seg, min(rr, rl + grp * seg + seg)
                    for col in range(ncol):
                        s = 4 + 4 * col
                        y0 = a + 4 * col - lev
                        for x in range(xa, xe):
                            pp = x - xs
                            R = [pl[prev][pp + d, s - 2:s + 4] for d in (-1, 0, 1)]
                            Rt = [plt[prev][pp + d, s - 2:s + 4] for d in (-1, 0, 1)]
                            o = []
                            for k in range(4):
                                y = y0 + k
                                if 1 <= y <= self.S2 - 2:
                                    need = tb + lev - 1
                                    for d in range(3):
                                        for e in range(3):
                                            yy = y + e - 1
                                            xx = x + d - 1
                                            ring = xx in (0, self.S1 - 1) or yy in (0, self.S2 - 1)
                                            t = Rt[d][k + e]
                                            if ring and 0 <= yy < self.S2 and R[d][k + e] != self.a[xx, yy]:
                                                raise AssertionError(
                                                    f"row m={r['m']} blk {b} j2 {j2} lev {lev} point ({x},{y}) "
                                                    f"ring ({xx},{yy}) holds {R[d][k + e]} tag {t}")
                                            if not ring and t != need:
                                                raise AssertionError(
                                                    f"row m={r['m']} blk {b} j2 {j2} lev {lev} point ({x},{y}) "
                                                    f"reads ({xx},{yy}) tag {t} need {need}")
                                    o.append(self.f(R, k))
                                elif y == 0 or y == self.S2 - 1:
                                    o.append(float(self.a[x, y]))
                                else:
                                    o.append(0.0)
                            new.append((pp, s, o, x, y0))
                            if self.is_facet(x, nl, nr, tb + lev == self.T):
                                for k in range(4):
                                    y = y0 + k
                                    if 1 <= y <= self.S2 - 2:
                                        self.gwrite(tb + lev, x, y, o[k])
                for pp, s, o, x, y0 in new:
                    for k in range(4):
                        pl[cur][pp, s + k] = o[k]
                        y = y0 + k
                        plt[cur][pp, s + k] = tb + lev if (1 <= y <= self.S2 - 2) else -2


def reference(a, T):
    w = np.array([[1 / 16, 1 / 8, 1 / 16], [1 / 8, 1 / 4, 1 / 8], [1 / 16, 1 / 8, 1 / 16]])
    b = a.astype(np.float64).copy()
    for _ in range(T):
        c = b.copy()
        S1, S2 = b.shape
        acc = np.zeros((S1 - 2, S2 - 2))
        for d1 in range(3):
            for d2 in range(3):
                acc += w[d1, d2] * b[d1:S1 - 2 + d1, d2:S2 - 2 + d2]
        c[1:-1, 1:-1] = acc
        b = c
    return b
