"""Pins of the CPU stencil oracle (oracle/stencil_oracle.c) to things other
than itself: hand values, a structurally different brute-force recursion,
exact fp64 linear algebra, closed-form Fourier symbols of Eq. 1's operator,
exact invariants and thread determinism.  PAPER.md §3, Eq. 1 (L352-366)
defines the iteration; R1-R4 fix the stencil bodies, the ring and
the expression order.  No GPU needed."""
from fractions import Fraction

import math
import numpy as np
import pytest

import oracle
from oracle import (FUSED, GRADIENT2D, HEAT2D_9PT, HEAT3D_7PT, JACOBI2D_5PT, LAPLACIAN2D_5PT,
                    LAPLACIAN3D_27PT, PLAIN)
from synth import field

LINEAR = [JACOBI2D_5PT, HEAT2D_9PT, LAPLACIAN2D_5PT, HEAT3D_7PT, LAPLACIAN3D_27PT]
ALL = LINEAR + [GRADIENT2D]
F32 = np.float32


# ------------------------------------------------------------------ exact fp32 helpers

def f32_round(q: Fraction) -> np.float32:
    """Nearest fp32 to the rational q, ties to even (used for an exact fmaf)."""
    f = np.float32(float(q))
    cands = [np.nextafter(f, F32(-np.inf)), f, np.nextafter(f, F32(np.inf))]

    def key(c):
        lsb = int(np.frombuffer(np.float32(c).tobytes(), np.uint32)[0]) & 1
        return (abs(Fraction(float(c)) - q), lsb)
    return F32(min(cands, key=key))


def fma32(a, b, c) -> np.float32:
    return f32_round(Fraction(float(a)) * Fraction(float(b)) + Fraction(float(c)))


# ------------------------------------------------------------------ T = 1 hand values

def test_T0_is_identity():
    for kind in ALL:
        dims = (7, 9) if oracle.KIND_NDIMS[kind] == 2 else (5, 6, 7)
        a = field(11, dims)
        for mode in (PLAIN, FUSED):
            assert np.array_equal(oracle.run(kind, a, 0, mode), a)


@pytest.mark.parametrize("mode", [PLAIN, FUSED])
def test_hand_values_2d(mode):
    g = np.arange(1, 10, dtype=np.float32).reshape(3, 3)
    # Jacobi 0.2*(2+4+5+6+8) = 5; Heat (1+3+7+9)/16 + (2+4+6+8)/8 + 5/4 = 5;
    # Laplacian-2D 5/2 + 20/8 = 5 (all exactly representable, R1)
    for kind in (JACOBI2D_5PT, HEAT2D_9PT, LAPLACIAN2D_5PT):
        out = oracle.run(kind, g, 1, mode)
        assert out[1, 1] == F32(5.0), (kind, out[1, 1])
        mask = np.ones_like(g, bool)
        mask[1, 1] = False
        assert np.array_equal(out[mask], g[mask])   # ring untouched


@pytest.mark.parametrize("mode", [PLAIN, FUSED])
def test_hand_values_3d(mode):
    g = np.arange(27, dtype=np.float32).reshape(3, 3, 3)
    # centre 13; faces sum 78, edges 156, corners 104:
    # Heat-3D 13/4 + 78/8 = 13; Laplacian-27 13/2 + 78*7/128 + 156*3/256 + 104/256 = 13
    for kind in (HEAT3D_7PT, LAPLACIAN3D_27PT):
        out = oracle.run(kind, g, 1, mode)
        assert out[1, 1, 1] == F32(13.0), (kind, out[1, 1, 1])


@pytest.mark.parametrize("mode", [PLAIN, FUSED])
def test_hand_value_gradient(mode):
    # n=1, s=2, w=1, e=1, c=4: gx=0, gy=0.5, g2=1.25, lap=-11,
    # out = 4 - (11/8)/sqrt(1.25) = 2.77016261237...
    g = np.array([[0, 1, 0], [1, 4, 1], [0, 2, 0]], dtype=np.float32)
    out = oracle.run(GRADIENT2D, g, 1, mode)[1, 1]
    exact = 4.0 - (11.0 / 8.0) / np.sqrt(1.25)
    assert abs(float(out) - exact) <= 2 * np.spacing(F32(exact))


def test_default_weights_match_readings():
    """DESIGN.md R1: the weights, and their closed-form Fourier symbols."""
    expect_sym = {
        JACOBI2D_5PT: lambda t: 0.2 * (1 + 2 * np.cos(t[0]) + 2 * np.cos(t[1])),
        HEAT2D_9PT: lambda t: np.cos(t[0] / 2) ** 2 * np.cos(t[1] / 2) ** 2,
        LAPLACIAN2D_5PT: lambda t: 0.5 + 0.25 * (np.cos(t[0]) + np.cos(t[1])),
        HEAT3D_7PT: lambda t: 0.25 + 0.25 * (np.cos(t[0]) + np.cos(t[1]) + np.cos(t[2])),
        LAPLACIAN3D_27PT: lambda t: (0.5 + (7 / 64) * np.sum(np.cos(t))
                                     + (3 / 64) * (np.cos(t[0]) * np.cos(t[1]) + np.cos(t[0]) * np.cos(t[2])
                                                   + np.cos(t[1]) * np.cos(t[2]))
                                     + (1 / 32) * np.prod(np.cos(t))),
    }
    rng = np.random.default_rng(0)
    for kind, sym in expect_sym.items():
        offs, w = oracle.stencil_info(kind)
        D = oracle.KIND_NDIMS[kind]
        assert len(w) == {1: 5, 2: 9, 6: 5, 4: 7, 5: 27}[kind]
        # canonical order is lexicographic over the offsets
        assert [tuple(o) for o in offs] == sorted(tuple(o) for o in offs)
        for _ in range(20):
            th = rng.uniform(0, np.pi, 3)[:D]
            got = sum(float(wj) * np.prod(np.cos(th * o[:D])) for o, wj in zip(offs, w))
            tol = 1e-7 if kind == JACOBI2D_5PT else 1e-14   # 0.2f is not 0.2
            assert abs(got - sym(th)) < tol, kind


# ------------------------------------------------------------------ brute force

def brute_force(kind, grid, T, mode):
    """Memoised top-down recursion of Eq. 1, structurally unlike the oracle's
    two-plane loop: value(t, s) is computed on demand from value(t-1, s+a)."""
    offs, w = oracle.stencil_info(kind)
    D = grid.ndim
    shape = grid.shape
    memo = {}

    def ring(idx):
        return any(i == 0 or i == n - 1 for i, n in zip(idx, shape))

    def val(t, idx):
        if t == 0 or ring(idx):
            return F32(grid[idx])
        key = (t, idx)
        if key in memo:
            return memo[key]
        if kind == GRADIENT2D:
            i, j = idx
            n, s = val(t - 1, (i - 1, j)), val(t - 1, (i + 1, j))
            we, e, c = val(t - 1, (i, j - 1)), val(t - 1, (i, j + 1)), val(t - 1, idx)
            gx = F32(0.5) * (e - we)
            gy = F32(0.5) * (s - n)
            if mode == FUSED:
                g2 = fma32(gy, gy, fma32(gx, gx, F32(1.0)))
            else:
                g2 = (F32(1.0) + gx * gx) + gy * gy
            lap = ((n - c) + (s - c)) + ((e - c) + (we - c))
            r = c + (F32(w[0]) * lap) / np.sqrt(g2)
        else:
            terms = [(F32(wj), val(t - 1, tuple(ii + int(o) for ii, o in zip(idx, oo[:D]))))
                     for oo, wj in zip(offs, w)]
            acc = terms[0][0] * terms[0][1]
            for wj, x in terms[1:]:
                acc = fma32(wj, x, acc) if mode == FUSED else acc + wj * x
        memo[key] = F32(r if kind == GRADIENT2D else acc)
        return memo[key]

    out = np.empty_like(grid)
    for idx in np.ndindex(*shape):
        out[idx] = val(T, idx)
    return out


@pytest.mark.parametrize("kind", ALL)
@pytest.mark.parametrize("mode", [PLAIN, FUSED])
def test_brute_force_bit_exact(kind, mode):
    D = oracle.KIND_NDIMS[kind]
    dims = (8, 8) if D == 2 else (6, 6, 6)
    Ts = (0, 1, 2, 3, 7, 8) if D == 2 else (0, 1, 2, 5)
    a = field(100 + kind, dims)
    for T in Ts:
        got = oracle.run(kind, a, T, mode)
        exp = brute_force(kind, a, T, mode)
        assert np.array_equal(got.view(np.uint32), exp.view(np.uint32)), (kind, mode, T)


# ------------------------------------------------------------------ exact linear algebra

def iteration_matrix(kind, shape):
    offs, w = oracle.stencil_info(kind)
    n = int(np.prod(shape))
    M = np.zeros((n, n))
    D = len(shape)
    for idx in np.ndindex(*shape):
        r = np.ravel_multi_index(idx, shape)
        if any(i == 0 or i == s - 1 for i, s in zip(idx, shape)):
            M[r, r] = 1.0
            continue
        for o, wj in zip(offs, w):
            q = tuple(i + int(d) for i, d in zip(idx, o[:D]))
            M[r, np.ravel_multi_index(q, shape)] += float(wj)
    return M


@pytest.mark.parametrize("kind", LINEAR)
def test_dense_iteration_matrix(kind):
    D = oracle.KIND_NDIMS[kind]
    shape = (9, 10) if D == 2 else (5, 6, 5)
    T = 16 if D == 2 else 8
    a = field(7, shape)
    M = iteration_matrix(kind, shape)
    x = a.astype(np.float64).ravel()
    for _ in range(T):
        x = M @ x
    nN = len(oracle.stencil_info(kind)[1])
    tol = 4 * T * nN * 2.0 ** -24 * np.abs(a).max()
    for mode in (PLAIN, FUSED):
        got = oracle.run(kind, a, T, mode).astype(np.float64).ravel()
        assert np.max(np.abs(got - x)) <= tol, (kind, mode)


@pytest.mark.parametrize("kind,dims,T,modes", [
    (JACOBI2D_5PT, (256, 256), 64, [(10, 10), (3, 7)]),            # C1 shape
    (JACOBI2D_5PT, (40, 40), 6, [(38, 37)]),                       # negative symbol
    (HEAT2D_9PT, (130, 70), 40, [(4, 5), (9, 2)]),
    (LAPLACIAN2D_5PT, (66, 66), 30, [(5, 6)]),
    (HEAT3D_7PT, (34, 30, 38), 20, [(2, 3, 4)]),
    (LAPLACIAN3D_27PT, (30, 34, 26), 16, [(3, 2, 5)]),
])
def test_fourier_mode_decay(kind, dims, T, modes):
    """A single sine mode with a zero ring is an eigenvector of the symmetric
    operator: u_T = lambda^T u_0 with lambda = sum_a w_a prod_d cos(theta_d a_d)."""
    offs, w = oracle.stencil_info(kind)
    D = len(dims)
    for p in modes:
        th = np.array([np.pi * p[d] / (dims[d] - 1) for d in range(D)])
        u = np.ones(dims)
        for d in range(D):
            s = np.sin(th[d] * np.arange(dims[d]))
            s[0] = s[-1] = 0.0
            u = u * s.reshape([-1 if e == d else 1 for e in range(D)])
        lam = sum(float(wj) * np.prod(np.cos(th * o[:D])) for o, wj in zip(offs, w))
        if lam < 0:
            assert T < 10
        u32 = u.astype(np.float32)
        tol = (4 * T * len(w) + 2) * 2.0 ** -24 * np.abs(u).max()
        for mode in (PLAIN, FUSED):
            got = oracle.run(kind, u32, T, mode).astype(np.float64)
            assert np.max(np.abs(got - lam ** T * u)) <= tol, (kind, p, mode, lam)


@pytest.mark.parametrize("kind", [HEAT2D_9PT, LAPLACIAN2D_5PT, HEAT3D_7PT, LAPLACIAN3D_27PT,
                                  GRADIENT2D, JACOBI2D_5PT])
def test_affine_fields_are_fixed_points(kind):
    """Symmetric weights summing to 1 map an affine field to itself; with
    dyadic weights and small-integer values every operation is exact, so the
    result is bit-identical for all T (Gradient: every difference is exact and
    lap = 0).  Jacobi uses dyadic coefficients passed through `coeffs`."""
    D = oracle.KIND_NDIMS[kind]
    dims = (12, 17) if D == 2 else (7, 8, 9)
    idx = np.indices(dims)
    coef = (3, -5, 7)[:D]
    a = (100 + sum(c * i for c, i in zip(coef, idx))).astype(np.float32)
    coeffs = None
    if kind == JACOBI2D_5PT:
        coeffs = [0.125, 0.125, 0.5, 0.125, 0.125]
    for mode in (PLAIN, FUSED):
        for T in (1, 5, 16):
            assert np.array_equal(oracle.run(kind, a, T, mode, coeffs=coeffs), a), (kind, mode, T)


def test_constant_c_term():
    """Eq. 1's +c: with c the field gains c each step in the interior (exact here)."""
    a = np.full((6, 7), 2.0, np.float32)
    offs, w = oracle.stencil_info(HEAT2D_9PT)
    coeffs = list(w) + [0.5]
    out = oracle.run(HEAT2D_9PT, a, 1, PLAIN, coeffs=coeffs)
    assert out[2, 3] == F32(2.5) and out[0, 0] == F32(2.0)


@pytest.mark.parametrize("kind", LINEAR)
def test_superposition(kind):
    D = oracle.KIND_NDIMS[kind]
    dims = (20, 23) if D == 2 else (9, 10, 11)
    x, y = field(1, dims), field(2, dims)
    T = 7
    lhs = oracle.run(kind, (0.5 * x + 0.25 * y).astype(np.float32), T).astype(np.float64)
    rhs = 0.5 * oracle.run(kind, x, T).astype(np.float64) + 0.25 * oracle.run(kind, y, T).astype(np.float64)
    assert np.max(np.abs(lhs - rhs)) < 1e-5


@pytest.mark.parametrize("kind", ALL)
def test_max_principle(kind):
    D = oracle.KIND_NDIMS[kind]
    dims = (31, 29) if D == 2 else (11, 12, 10)
    a = field(5, dims)
    out = oracle.run(kind, a, 12)
    ulp = 8 * 2.0 ** -24
    assert out.min() >= a.min() - ulp and out.max() <= a.max() + ulp


@pytest.mark.parametrize("kind", ALL)
def test_thread_count_determinism(kind):
    D = oracle.KIND_NDIMS[kind]
    dims = (67, 45) if D == 2 else (19, 17, 21)
    a = field(9, dims)
    for mode in (PLAIN, FUSED):
        o1 = oracle.run(kind, a, 9, mode, nthreads=1)
        o4 = oracle.run(kind, a, 9, mode, nthreads=4)
        assert np.array_equal(o1, o4)


@pytest.mark.parametrize("kind", ALL)
def test_fused_vs_plain_within_1e5(kind):
    """BASELINE.json north_star: the contracted-FMA build stays within 1e-5 max
    relative error (reading R5) of the plain one after T steps."""
    D = oracle.KIND_NDIMS[kind]
    dims = (64, 80) if D == 2 else (20, 22, 24)
    a = field(3, dims)
    p = oracle.run(kind, a, 64, PLAIN).astype(np.float64)
    f = oracle.run(kind, a, 64, FUSED).astype(np.float64)
    rel = np.abs(f - p) / np.maximum(np.abs(p), 2.0 ** -10)
    assert rel.max() <= 1e-5


def test_rejects_bad_arguments():
    a = field(1, (8, 8))
    with pytest.raises(ValueError):
        oracle.run(HEAT3D_7PT, a, 1)          # ndims mismatch
    with pytest.raises(ValueError):
        oracle.run(HEAT2D_9PT, a, -1)
    with pytest.raises(ValueError):
        oracle.run(HEAT2D_9PT, a, 1, coeffs=[1.0, 2.0])


# ------------------------------------------------------------------ Jacobi-1D
# The 1D 3-point average the paper's derivation starts from (Eqs. 2-12);
# weights fp32(1/3) each (reading R1, PolyBench jacobi-1d), canonical order.

def test_jacobi1d_hand_values():
    # (3 + 6 + 9)/3: w*3 = 1.00000003 -> 1, w*6 -> 2 (+ 1 = 3), w*9 -> 3 (+ 3 = 6) in both modes
    g = np.array([3.0, 6.0, 9.0], np.float32)
    for mode in (PLAIN, FUSED):
        out = oracle.run(oracle.JACOBI1D_3PT, g, 1, mode)
        assert out[1] == F32(6.0) and out[0] == g[0] and out[2] == g[2], (mode, out)
    offs, w = oracle.stencil_info(oracle.JACOBI1D_3PT)
    assert [tuple(o) for o in offs] == [(-1, 0, 0), (0, 0, 0), (1, 0, 0)]
    assert all(x == F32(1.0) / F32(3.0) for x in w)


@pytest.mark.parametrize("mode", [PLAIN, FUSED])
def test_jacobi1d_brute_force_bit_exact(mode):
    a = field(107, (12,))
    for T in (0, 1, 2, 5, 9):
        got = oracle.run(oracle.JACOBI1D_3PT, a, T, mode)
        exp = brute_force(oracle.JACOBI1D_3PT, a, T, mode)
        assert np.array_equal(got.view(np.uint32), exp.view(np.uint32)), (mode, T)


def test_jacobi1d_dense_matrix_and_fourier():
    kind = oracle.JACOBI1D_3PT
    a = field(9, (40,))
    M = iteration_matrix(kind, (40,))
    x = a.astype(np.float64)
    for _ in range(30):
        x = M @ x
    for mode in (PLAIN, FUSED):
        got = oracle.run(kind, a, 30, mode).astype(np.float64)
        assert np.max(np.abs(got - x)) <= 4 * 30 * 3 * 2.0 ** -24
    # sine mode with a zero ring: u_T = lambda^T u_0, lambda = w (1 + 2 cos theta)
    n, p, T = 101, 7, 50
    th = np.pi * p / (n - 1)
    u = np.sin(th * np.arange(n))
    u[0] = u[-1] = 0.0
    w = float(F32(1.0) / F32(3.0))
    lam = w * (1 + 2 * np.cos(th))
    for mode in (PLAIN, FUSED):
        got = oracle.run(kind, u.astype(np.float32), T, mode).astype(np.float64)
        assert np.max(np.abs(got - lam ** T * u)) <= (4 * T * 3 + 2) * 2.0 ** -24


def test_jacobi1d_fused_vs_plain_and_threads():
    a = field(5, (5001,))
    p = oracle.run(oracle.JACOBI1D_3PT, a, 64, PLAIN)
    f = oracle.run(oracle.JACOBI1D_3PT, a, 64, FUSED)
    assert np.max(np.abs(f.astype(np.float64) - p) / np.maximum(np.abs(p), 2.0 ** -10)) <= 1e-5
    assert np.array_equal(oracle.run(oracle.JACOBI1D_3PT, a, 64, FUSED, nthreads=1), f)


# ---- radius-r 1D binomial smoothers (kinds 8-10)
@pytest.mark.parametrize("kind,R", [(8, 2), (9, 3), (10, 4)])
def test_radius_r_hand_values_and_ring(kind, R):
    """T = 1 by hand: binomial weights C(2R, k)/4^R on x^2 give
    E[(x+D)^2] = x^2 + Var(D) = x^2 + R/2 exactly (D = centred Binomial(2R, 1/2));
    the ring (R cells each side) is untouched."""
    a = (np.arange(3 * R + 8, dtype=np.float32)) ** 2
    out = oracle.run(kind, a, 1, oracle.FUSED)
    x = np.arange(a.size, dtype=np.float64)
    inner = slice(R, a.size - R)
    assert np.array_equal(out[inner], (x ** 2 + R / 2.0)[inner].astype(np.float32))
    assert np.array_equal(out[:R], a[:R]) and np.array_equal(out[-R:], a[-R:])
    offs, w = oracle.stencil_info(kind)
    assert offs[:, 0].tolist() == list(range(-R, R + 1))
    assert np.array_equal(w.astype(np.float64) * 4 ** R, [math.comb(2 * R, k) for k in range(2 * R + 1)])


@pytest.mark.parametrize("kind,R", [(8, 2), (9, 3), (10, 4)])
def test_radius_r_fourier_mode(kind, R):
    """Binomial smoothing has the closed-form symbol lambda = cos(theta/2)^(2R):
    a sine mode vanishing on the ring decays by lambda^T (the ring of width R
    holds the mode's exact values, which equal the periodic continuation only
    at the zero-crossings, so the comparison stays outside the ring's cone of
    influence, R*T cells from each end)."""
    S, T = 4001, 40
    p = 400
    th = math.pi * p / (S - 1)
    x = np.arange(S)
    u0 = np.sin(th * x).astype(np.float32)
    lam = math.cos(th / 2) ** (2 * R)
    got = oracle.run(kind, u0, T, oracle.FUSED).astype(np.float64)
    # points farther than R*T from both ends only see the sine (odd extension of
    # sin(theta x) about x = 0 and x = S-1 continues it exactly)
    core = slice(R * T + R, S - R * T - R)
    assert np.max(np.abs(got[core] - lam ** T * np.sin(th * x[core]))) <= (4 * T * (2 * R + 1) + 2) * 2.0 ** -24
    assert lam ** T < 0.5                          # the identity map would fail the check above


@pytest.mark.parametrize("kind,R", [(8, 2), (10, 4)])
def test_radius_r_dense_matrix_and_affine(kind, R):
    """Independent check of the loop: a dense fp64 iteration matrix (ring rows
    identity), x_T = M^T x_0 within 4 T |N| 2^-24 max|x|; and an affine field
    with short mantissas is an exact fixed point (symmetric dyadic weights)."""
    from synth import field
    S, T = 23, 7
    a = field(5, (S,))
    offs, w = oracle.stencil_info(kind)
    M = np.eye(S)
    for i in range(R, S - R):
        M[i, :] = 0.0
        for o, wj in zip(offs[:, 0], w.astype(np.float64)):
            M[i, i + o] += wj
    ref = np.linalg.matrix_power(M, T) @ a.astype(np.float64)
    got = oracle.run(kind, a, T, oracle.FUSED).astype(np.float64)
    assert np.max(np.abs(got - ref)) <= 4 * T * len(w) * 2.0 ** -24 * np.max(np.abs(a))
    aff = (3.0 + 2.0 * np.arange(S)).astype(np.float32)
    assert np.array_equal(oracle.run(kind, aff, T, oracle.PLAIN), aff)
