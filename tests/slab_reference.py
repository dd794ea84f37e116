"""Reference implementation of the multi-GPU slab algorithm in
torch, TEST INFRASTRUCTURE ONLY: the gloo tests (tests/test_dist.py) run it
with the CPU oracle as the per-tile stepper and compare the gathered owned rows
with the single-domain oracle, which pins the algorithm the product implements
in C++ (paper_conf_ppopp_prajapatirradg17_b200/csrc/hhc_dist.cu:
stencil_run_dist); the product's partition is checked against `partition`
here (tests/test_dist.py)."""
from __future__ import annotations

from dataclasses import dataclass


@dataclass
class Slab:
    rank: int
    world: int
    S1: int
    own: int        # interior rows per rank (last rank may own fewer)
    r0: int         # first owned interior row
    r1: int         # one past the last owned interior row
    e0: int         # first row of the ghost-extended slab
    e1: int         # one past the last row of the extended slab
    g: int          # ghost depth (= tT)

    @property
    def rows(self) -> int:
        return self.e1 - self.e0

    @property
    def held(self):
        """Rows of the global grid the rank's in/out slab holds: the owned
        rows plus the physical ring row on the edge ranks."""
        lo = self.r0 - (1 if self.rank == 0 else 0)
        hi = self.r1 + (1 if self.rank == self.world - 1 else 0)
        return lo, hi


def partition(S1: int, world: int, rank: int, g: int) -> Slab:
    interior = S1 - 2
    own = -(-interior // world)
    r0 = 1 + rank * own
    r1 = min(1 + (rank + 1) * own, S1 - 1)
    if r1 <= r0:
        raise ValueError(f"rank {rank} owns no rows (S1={S1}, world={world})")
    if world > 1 and own < g:
        raise ValueError(f"slab of {own} rows is thinner than the ghost depth {g}: use a smaller tT")
    if world > 1 and r1 - r0 < g and rank < world - 1:
        raise ValueError("slab thinner than the ghost depth")
    e0 = max(0, r0 - g)
    e1 = min(S1, r1 + g)
    return Slab(rank, world, S1, own, r0, r1, e0, e1, g)


def exchange(slab: Slab, plane, xp_dist):
    """Fill the ghost rows of `plane` (the extended slab, rows e0..e1) from the
    neighbours' owned rows.  `xp_dist` is torch.distributed."""
    import torch
    ops = []
    g = slab.g
    lo = slab.r0 - slab.e0          # local index of the first owned row
    hi = slab.r1 - slab.e0          # local index one past the last owned row
    if slab.rank > 0:
        up_send = plane[lo:lo + g]
        up_recv = plane[lo - g:lo]
        ops.append(xp_dist.P2POp(xp_dist.isend, up_send.contiguous(), slab.rank - 1))
        ops.append(xp_dist.P2POp(xp_dist.irecv, up_recv, slab.rank - 1))
    if slab.rank < slab.world - 1:
        dn_send = plane[hi - g:hi]
        dn_recv = plane[hi:hi + g]
        ops.append(xp_dist.P2POp(xp_dist.isend, dn_send.contiguous(), slab.rank + 1))
        ops.append(xp_dist.P2POp(xp_dist.irecv, dn_recv, slab.rank + 1))
    if ops:
        for r in xp_dist.batch_isend_irecv(ops):
            r.wait()
    return torch


def run_slabs(slab: Slab, plane0, plane1, T: int, tT: int, stepper, xp_dist):
    """Drive the time tiles.  plane0 holds level 0 of the extended slab (ring and
    ghosts included); stepper(plane0, plane1, Tt) runs Tt steps leaving the
    result in plane0 (Tt even) or plane1 (Tt odd).  Returns the plane holding A_T."""
    done = 0
    cur = plane0
    while done < T:
        Tt = min(tT, T - done)
        if slab.world > 1:
            exchange(slab, cur, xp_dist)
        out = stepper(cur, plane1 if cur is plane0 else plane0, Tt)
        cur = out
        done += Tt
    return cur


def run_slabs_overlap(slab: Slab, plane0, plane1, T: int, tT: int, stepper_int, stepper_edge, xp_dist,
                      streams=None):
    """The time-tile loop with the exchange overlapped (SURVEY §8(e) "Overlap").

    Per tile: the two edge sub-slabs -- 3g rows around each neighbour side, fresh
    ghosts included -- run first (stepper_edge, second stream) and their exact
    owned rows [lo, lo+g) / [hi-g, hi) are sent to the neighbours at once; the
    interior sub-slab (the owned rows alone, whose edge rows act as a fixed ring
    for the tile) needs no ghosts and runs concurrently (stepper_int, first
    stream).  After tT <= g steps the interior run is exact on [lo+g, hi-g), the
    edge runs on the g rows next to each side (dependence cone of tT rows), so
    the tile's result is the interior plane with the edge rows and the received
    ghosts written in.  Redundant work: 3g rows per neighbour side per tile.

    `streams` = (s1, s2) torch.cuda streams, or None (CPU: sequential).  Falls
    back to run_slabs when a slab is thinner than 2g rows."""
    import torch
    g = slab.g
    lo, hi = slab.r0 - slab.e0, slab.r1 - slab.e0
    up, dn = slab.rank > 0, slab.rank < slab.world - 1
    if not (up or dn) or hi - lo < 2 * g:
        return run_slabs(slab, plane0, plane1, T, tT, stepper_int, xp_dist)
    A, B = (lo if up else 0), (hi if dn else slab.rows)
    tail = tuple(plane0.shape[1:])

    def buf(n):
        return torch.empty((n,) + tail, dtype=plane0.dtype, device=plane0.device)

    e_up = (lo - g, lo + 2 * g) if up else None          # local rows of the edge sub-slabs
    e_dn = (hi - 2 * g, hi + g) if dn else None
    t_bufs = (buf(3 * g), buf(3 * g)) if up else None
    b_bufs = (buf(3 * g), buf(3 * g)) if dn else None
    r_up = buf(g) if up else None
    r_dn = buf(g) if dn else None
    s1, s2 = streams if streams is not None else (None, None)

    def on(st):
        return torch.cuda.stream(st) if st is not None else _Null()

    exchange(slab, plane0, xp_dist)                      # ghosts of tile 0 (blocking)
    cur, oth = plane0, plane1
    done = 0
    while done < T:
        Tt = min(tT, T - done)
        last = done + Tt >= T
        with on(s1):                                     # edge inputs taken before the interior overwrites cur
            if up:
                t_bufs[0].copy_(cur[e_up[0]:e_up[1]])
            if dn:
                b_bufs[0].copy_(cur[e_dn[0]:e_dn[1]])
        if s2 is not None:
            s2.wait_stream(s1)
        works = []
        with on(s2):
            te = stepper_edge(t_bufs[0], t_bufs[1], Tt) if up else None
            be = stepper_edge(b_bufs[0], b_bufs[1], Tt) if dn else None
            if not last:
                ops = []
                if up:
                    ops.append(xp_dist.P2POp(xp_dist.isend, te[g:2 * g], slab.rank - 1))
                    ops.append(xp_dist.P2POp(xp_dist.irecv, r_up, slab.rank - 1))
                if dn:
                    ops.append(xp_dist.P2POp(xp_dist.isend, be[g:2 * g], slab.rank + 1))
                    ops.append(xp_dist.P2POp(xp_dist.irecv, r_dn, slab.rank + 1))
                works = xp_dist.batch_isend_irecv(ops)
        with on(s1):
            stepper_int(cur[A:B], oth[A:B], Tt)           # overlaps the exchange
            res = cur if Tt % 2 == 0 else oth
            if s2 is not None:
                s1.wait_stream(s2)
            for w in works:
                w.wait()
            if up:
                res[lo:lo + g].copy_(te[g:2 * g])
                if not last:
                    res[lo - g:lo].copy_(r_up)
            if dn:
                res[hi - g:hi].copy_(be[g:2 * g])
                if not last:
                    res[hi:hi + g].copy_(r_dn)
        cur, oth = res, (plane1 if res is plane0 else plane0)
        done += Tt
    return cur


class _Null:
    def __enter__(self):
        return self

    def __exit__(self, *a):
        return False


