"""CPU mirror of the K1P kernel (hex2d_pair_kernel, csrc/hhc_kernels_pair.cu):
same schedule, planes, face, stage, footprint and per-lane column layout, with
the warps of a pass executed one after the other (no cross-warp dependence
inside a pass by design) and lanes vectorised.  Used to localise logic bugs
on CPU; a linear 9-point stencil in float64 replaces the kernel arithmetic.
Test infrastructure only."""
from __future__ import annotations

import numpy as np

from sim_hex2d import plan_rows, cdiv

W9 = np.array([[1 / 16, 1 / 8, 1 / 16], [1 / 8, 1 / 4, 1 / 8], [1 / 16, 1 / 8, 1 / 16]])


def point(r0, r1, r2, k):
    rows = (r0, r1, r2)
    return sum(W9[d1][d2] * rows[d1][k + d2] for d1 in range(3) for d2 in range(3))


class SimPair:
    CW = 124

    def __init__(self, a, T, tile, G=1):
        self.a = a.astype(np.float64)
        self.S1, self.S2 = a.shape
        self.T = T
        self.tT, self.tS1, self.tS2 = tile[:3]
        assert self.tS2 % self.CW == 0
        self.nw = self.tS2 // self.CW
        self.G = G
        self.plane = [self.a.copy(), np.full(a.shape, np.nan)]
        ring = np.zeros(a.shape, bool)
        ring[0, :] = ring[-1, :] = ring[:, 0] = ring[:, -1] = True
        self.plane[1][ring] = self.a[ring]

    # ---- geometry (mirror of build_geo) ----------------------------------------
    def hex_row(self, x0, lo, nlev, lev):
        if lev < 0 or lev >= nlev:
            return 0, 0
        tau = lo + lev
        mm = min(tau, self.tT - tau)
        l = max(x0 - mm, 1)
        r = min(x0 + self.tS1 + mm, self.S1 - 1)
        return (l, max(r, l))

    def geo(self, x0, xs, lo, nlev, tb):
        out = []
        for lev in range(nlev):
            rl, rr = self.hex_row(x0, lo, nlev, lev)
            pl, pr = self.hex_row(x0, lo, nlev, lev - 1)
            empty = rl >= rr
            A0, A1 = rl - 1, rr + 1
            first = lev == 0 or pl >= pr
            if first:
                f = (A0, A1, A1, A1, A1, A1)
            else:
                f1a, f1b = A0, max(A0, min(A1, pl))
                f2a, f2b = min(A1, max(pr, A0)), A1
                if f2a < f1b:
                    f2a = f1b
                ia, ib = max(A0, pl), min(A1, pr)
                ib = max(ib, ia)
                f = (f1a, f1b, f2a, f2b, ia, ib)
            nl, nr = self.hex_row(x0, lo, nlev, lev + 1)
            final = tb + lev == self.T
            if final or nl >= nr:
                gap = (0, 0)
            else:
                xl = xs - 4 if nl <= 1 else nl + 1
                xh = xs + (self.tS1 + self.tT + 2) + 4 if nr >= self.S1 - 1 else nr - 1
                gap = (0, 0) if xl >= xh else (max(xl - xs, -2), min(xh - xs, self.tS1 + self.tT + 4))
            seg = cdiv(rr - rl, self.G)
            out.append(dict(f=[v - xs for v in f], first=first, empty=empty, rl=rl - xs, rr=rr - xs,
                            gap=gap, seg=seg))
        return out

    def sched(self, geo, nlev):
        s = [None] * nlev
        k = 0
        l = 0
        while l < nlev:
            if l + 1 < nlev and not geo[l]["empty"] and not geo[l + 1]["empty"] and not geo[l + 1]["first"]:
                s[l] = (2, k)
                s[l + 1] = (0, k)
                l += 2
            else:
                s[l] = (1, k)
                l += 1
            k += 1
        return s

    def gget(self, t, x, y):
        v = self.plane[t & 1][x, y]
        assert not np.isnan(v), f"read of unwritten value level {t} at {(x, y)}"
        return v

    def run(self):
        for r in plan_rows((self.S1, self.S2), self.T, (self.tT, self.tS1, self.tS2)):
            for b in range(r["w"]):
                self.block(r, b)
        return self.plane[self.T & 1]

    def block(self, r, b):
        tT, tS1, tS2, G, nw = self.tT, self.tS1, self.tS2, self.G, self.nw
        S1, S2 = self.S1, self.S2
        NX = tS1 + tT + 2
        RS = tS2 + 8
        x0 = r["xbase"] + b * (2 * tS1 + tT)
        xs = x0 - tT // 2 - 1
        lo = r["lo"]
        nlev = r["hi"] - lo
        tb = r["t0"] + lo
        geo = self.geo(x0, xs, lo, nlev, tb)
        sched = self.sched(geo, nlev)
        # smem: planes with guard rows at index 0 and NX+1 (row pp stored at pp+1)
        pl = [np.full((NX + 2, RS), np.nan), np.full((NX + 2, RS), np.nan)]
        face = np.full((2, tT + 1, NX, 6), np.nan)
        stage = np.full((2, 4, tS2 + 4), np.nan)
        lanes = np.arange(32)
        for j2 in range(r["n2"]):
            a = 1 + j2 * tS2
            fc, fn = j2 & 1, (j2 + 1) & 1
            # ---- footprint
            W = tS2 + 6
            for l in range(nlev):
                g = geo[l]
                typ, k = sched[l]
                if g["empty"] or typ == 0:
                    continue
                halo_all = g["first"] or j2 == 0
                dpl = pl[(k + 1) & 1]
                ybase = a - 5 - l
                f = g["f"]
                segs = [(f[0], f[1], True), (f[2], f[3], True)] + ([(f[4], f[5], False)] if halo_all else [])
                for pa, pb, full in segs:
                    for pp in range(pa, pb):
                        x = xs + pp
                        if l > 0 and (x == 0 or x == S1 - 1):
                            continue
                        for c in range(W if full else 6):
                            if c < 6 and j2 > 0:
                                continue            # halo columns: from the face (previous sub-tile)
                            y = ybase + c
                            if y < 0 or y >= S2:
                                continue
                            v = self.gget(tb + l - 1, x, y)
                            if c >= 6 or l == 0:
                                dpl[pp + 1, c + 2] = v
                            else:
                                face[fc, l, pp, c] = v
            if j2 > 0:                                 # halo of the first pass from the face
                R0 = pl[(sched[0][1] + 1) & 1]
                for pp in range(NX):                   # ring rows included: the face holds them
                    R0[pp + 1, 2:8] = face[fc, 0, pp, :]
            if sched[0][0] == 2:
                self.load_stage(stage[0], geo[1], xs, a, 0, tb)
            npair = 0
            l = 0
            while l < nlev:
                typ, k = sched[l]
                R = pl[(k + 1) & 1]
                Wp = pl[k & 1]
                lout = l + 1 if typ == 2 else l
                g = geo[l]
                for pp in range(NX):
                    xr = xs + pp
                    face[fn, l, pp, :] = R[pp + 1, tS2 + 2:tS2 + 8]   # level l-1, last 6 columns
                    if lout + 1 < nlev and xr != 0 and xr != S1 - 1:
                        Wp[pp + 1, 2:8] = face[fc, lout + 1, pp, :]
                if xs <= 0 or xs + NX > S1 - 1:
                    for xr in (0, S1 - 1):
                        pp = xr - xs
                        if 0 <= pp < NX:
                            for slot in range(2, tS2 + 8):
                                y = a + slot - 8 - lout
                                Wp[pp + 1, slot] = self.a[xr, y] if 0 <= y < S2 else 0.0
                ln = lout + 1
                pending = None
                if ln + 1 < nlev and sched[ln][0] == 2:
                    pending = ((npair + (1 if typ == 2 else 0)) & 1, geo[ln + 1], ln)
                if not g["empty"]:
                    for grp in range(G):
                        for wgi in range(nw):
                            colbase = self.CW * wgi + 4 * lanes
                            if typ == 1:
                                self.single(l, g, grp, wgi, colbase, a, xs, R, Wp, face[fn], tb, RS, NX)
                            else:
                                self.pair(l, g, geo[l + 1], grp, wgi, colbase, a, xs, R, Wp, face[fn],
                                          stage[npair & 1], tb, RS, NX)
                if pending is not None:
                    self.load_stage(stage[pending[0]], pending[1], xs, a, pending[2], tb)
                if typ == 2:
                    npair += 1
                l += 2 if typ == 2 else 1

    def load_stage(self, st, gn, xs, a, ln, tb):
        f = gn["f"]
        slot = 0
        for seg in range(2):
            for X in range(f[2 * seg], f[2 * seg + 1]):
                x = xs + X
                if not (x == 0 or x == self.S1 - 1):
                    for c in range(self.tS2 + 4):
                        y = a - 4 + c - ln
                        if 0 <= y < self.S2:
                            st[slot, c] = self.gget(tb + ln, x, y)
                slot += 1

    def fix(self, o, x, y0):
        for k in range(4):
            y = y0 + k
            bad = (y < 1) | (y > self.S2 - 2)
            ring = (y == 0) | (y == self.S2 - 1)
            o[k] = np.where(ring, self.a[x, np.clip(y, 0, self.S2 - 1)], np.where(bad, 0.0, o[k]))
        return o

    def rows6(self, P, pp, s):
        return np.stack([P[pp + 1, s - 2 + j] for j in range(6)])      # [6][32]

    def single(self, l, g, grp, wgi, colbase, a, xs, R, Wp, fnxt, tb, RS, NX):
        seg = g["seg"]
        pa = g["rl"] + grp * seg
        pe = min(g["rr"], pa + seg)
        s = colbase + 4
        u0 = a - 4 + colbase
        y0 = u0 - l
        lanes = np.arange(32)
        for pp in range(pa, pe):
            r0, r1, r2 = self.rows6(R, pp - 1, s), self.rows6(R, pp, s), self.rows6(R, pp + 1, s)
            o = [point(r0, r1, r2, k) for k in range(4)]
            o = self.fix(o, xs + pp, y0)
            for L in range(1, 32):
                Wp[pp + 1, s[L]:s[L] + 4] = [o[k][L] for k in range(4)]
            nwlo, nwhi = g["gap"]
            if not (nwlo <= pp < nwhi):
                for L in range(1, 32):
                    for k in range(4):
                        y = y0[L] + k
                        if 1 <= y <= self.S2 - 2:
                            self.plane[(tb + l) & 1][xs + pp, y] = o[k][L]

    def pair(self, l, g, gn, grp, wgi, colbase, a, xs, R, Wp, fnxt, st, tb, RS, NX):
        G = self.G
        rl, rr = g["rl"], g["rr"]
        rln, rrn = gn["rl"], gn["rr"]
        segn = cdiv(rrn - rln, G)
        a1 = rln + grp * segn
        e1 = min(rrn, a1 + segn)
        if a1 >= e1:
            return
        own_lo = -1000 if grp == 0 else a1
        own_hi = 1000 if a1 + segn >= rrn else e1
        s = colbase + 4
        u0 = a - 4 + colbase
        y0 = u0 - l
        y1 = y0 - 1
        f = gn["f"]
        f1a, f1n, f2a = f[0], f[1] - f[0], f[2]
        Lm = np.zeros((6, 32))
        Lc = np.zeros((6, 32))
        for x in range(a1 - 1, e1 + 1):
            xg = xs + x
            if rl <= x < rr:
                r0, r1, r2 = self.rows6(R, x - 1, s), self.rows6(R, x, s), self.rows6(R, x + 1, s)
                o = [point(r0, r1, r2, k) for k in range(4)]
                o = self.fix(o, xg, y0)
                if own_lo <= x < own_hi:
                    nwlo, nwhi = g["gap"]
                    if not (nwlo <= x < nwhi):
                        for L in range(1, 32):
                            for k in range(4):
                                y = y0[L] + k
                                if 1 <= y <= self.S2 - 2:
                                    self.plane[(tb + l) & 1][xg, y] = o[k][L]
            elif xg == 0 or xg == self.S1 - 1:
                o = []
                for k in range(4):
                    y = y0 + k
                    o.append(np.where((y >= 0) & (y < self.S2), self.a[xg, np.clip(y, 0, self.S2 - 1)], 0.0))
            else:
                slot = x - f1a if (f1a <= x < f1a + f1n) else f1n + (x - f2a)
                o = [st[slot, colbase + k] for k in range(4)]
            Ln = np.zeros((6, 32))
            Ln[0, 1:] = o[2][:-1]
            Ln[1, 1:] = o[3][:-1]
            for k in range(4):
                Ln[2 + k] = o[k]
            xm = x - 1
            if xm >= a1:
                q = [point(Lm, Lc, Ln, k) for k in range(4)]
                q = self.fix(q, xs + xm, y1)
                for L in range(1, 32):
                    Wp[xm + 1, s[L]:s[L] + 4] = [q[k][L] for k in range(4)]
                nwlo, nwhi = gn["gap"]
                if not (nwlo <= xm < nwhi):
                    for L in range(1, 32):
                        for k in range(4):
                            y = y1[L] + k
                            if 1 <= y <= self.S2 - 2:
                                self.plane[(tb + l + 1) & 1][xs + xm, y] = q[k][L]
            Lm, Lc = Lc, Ln
