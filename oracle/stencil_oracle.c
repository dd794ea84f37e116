/*
 * oracle/stencil_oracle.c -- TEST INFRASTRUCTURE ONLY.
 *
 * Plain, slow, obviously-correct CPU oracle for the stencil iteration of
 * PAPER.md §3, Eq. 1 (L352-366):
 *
 *     A_t(s) = ( sum_{a in N} w_a * A_{t-1}(s + a) ) + c ,   s in S, t = 1..T
 *
 * with the initial value A_0 = `in` and fixed boundary values (the one-cell
 * ring of the array, reading R2).  HHC tiling (§3.1) only
 * reorders WHICH points are computed WHEN; it never changes the per-point
 * expression or its operands, so the tiled GPU result must equal this naive
 * two-plane time stepping bit for bit once the per-point expression order is
 * fixed (reading R4, "canonical expression").
 *
 * Only tests/, __graft_entry__.smoke() and bench.py (cpu_baseline leg,
 * --impl reference) may load this library.  It shares no code, header, table
 * or constant with the CUDA path (paper_conf_ppopp_prajapatirradg17_b200/csrc).
 *
 * Build (see oracle/__init__.py): gcc -O2 -ffp-contract=off -fno-fast-math
 *        -fopenmp -shared -fPIC.  -ffp-contract=off keeps `acc + w*x` as a
 * separately rounded multiply and add ("plain" mode); "fused" mode calls
 * fmaf() explicitly.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <omp.h>

/* Stencil kinds (numbering is part of the C ABI contract in include/hhc.h,
 * re-declared here on purpose: the oracle includes nothing from the product). */
enum { O_JACOBI1D_3PT = 7,
       O_JACOBI2D_5PT = 1, O_HEAT2D_9PT = 2, O_GRADIENT2D = 3,
       O_HEAT3D_7PT = 4, O_LAPLACIAN3D_27PT = 5, O_LAPLACIAN2D_5PT = 6,
       /* SURVEY §8(f) f4, higher-order stencils ("Generality"):
        * 1D radius-r binomial smoothers, r = 2, 3, 4 */
       O_BINOM1D_R2 = 8, O_BINOM1D_R3 = 9, O_BINOM1D_R4 = 10 };
enum { O_MODE_PLAIN = 0, O_MODE_FUSED = 1 };

typedef struct {
    int ndims;
    int n;              /* |N| */
    int off[27][3];     /* offsets (d1,d2,d3), lexicographic over {-1,0,1}^D */
    float w[27];
    int has_c;
    float c;
    int gradient;
    float kappa;
} o_stencil;

static int o_kind_ndims(int kind) {
    switch (kind) {
    case O_JACOBI2D_5PT: case O_HEAT2D_9PT: case O_GRADIENT2D: case O_LAPLACIAN2D_5PT: return 2;
    case O_HEAT3D_7PT: case O_LAPLACIAN3D_27PT: return 3;
    case O_JACOBI1D_3PT: case O_BINOM1D_R2: case O_BINOM1D_R3: case O_BINOM1D_R4: return 1;
    default: return 0;
    }
}

/* Radius of the neighbourhood: 1, or r for the f4 kinds (offsets -r..r). */
static int o_kind_radius(int kind) {
    return kind == O_BINOM1D_R2 ? 2 : kind == O_BINOM1D_R3 ? 3 : kind == O_BINOM1D_R4 ? 4 : 1;
}

/* Is offset (number of non-zero components = nz) in N_kind? */
static int o_in_neigh(int kind, int nz) {
    switch (kind) {
    case O_JACOBI2D_5PT: case O_LAPLACIAN2D_5PT: case O_HEAT3D_7PT: case O_GRADIENT2D:
        return nz <= 1;                        /* centre + faces */
    case O_HEAT2D_9PT: case O_LAPLACIAN3D_27PT: case O_JACOBI1D_3PT:
        return 1;                              /* full 3^D box */
    default: return 0;
    }
}

/* Default weights (reading R1; the paper prints no stencil body,
 * PAPER.md L1175-1178), indexed by the number of non-zero offset components. */
static float o_default_weight(int kind, int nz) {
    switch (kind) {
    case O_JACOBI2D_5PT: return 0.2f;
    case O_JACOBI1D_3PT: return 1.0f / 3.0f;   /* PolyBench jacobi-1d averaging, fp32(1/3) */
    case O_LAPLACIAN2D_5PT: return nz == 0 ? 0.5f : 0.125f;
    case O_HEAT2D_9PT: return nz == 0 ? 0.25f : (nz == 1 ? 0.125f : 0.0625f);
    case O_HEAT3D_7PT: return nz == 0 ? 0.25f : 0.125f;
    case O_LAPLACIAN3D_27PT:
        return nz == 0 ? 0.5f : nz == 1 ? 7.0f / 128.0f : nz == 2 ? 3.0f / 256.0f : 1.0f / 256.0f;
    default: return 0.0f;
    }
}

static int o_build(int kind, const float* coeffs, int ncoeffs, o_stencil* s) {
    memset(s, 0, sizeof(*s));
    s->ndims = o_kind_ndims(kind);
    if (s->ndims == 0) return -1;
    if (kind == O_GRADIENT2D) {
        s->gradient = 1;
        s->kappa = 0.125f;
        if (coeffs) {
            if (ncoeffs != 1) return -1;
            s->kappa = coeffs[0];
        }
        return 0;
    }
    int D = s->ndims;
    int r = o_kind_radius(kind);
    if (r > 1) {
        /* binomial weights C(2r, k) / 4^r on the offsets -r..r (dyadic, positive, sum 1) */
        double c = 1.0, den = 1.0;
        for (int k = 0; k < 2 * r; ++k) den *= 2.0;
        for (int k = 0; k <= 2 * r; ++k) {
            s->off[s->n][0] = k - r; s->off[s->n][1] = 0; s->off[s->n][2] = 0;
            s->w[s->n] = (float)(c / den);
            s->n++;
            c = c * (double)(2 * r - k) / (double)(k + 1);
        }
    } else {
    int lo3 = (D == 3) ? -1 : 0, hi3 = (D == 3) ? 1 : 0;
    int lo2 = (D >= 2) ? -1 : 0, hi2 = (D >= 2) ? 1 : 0;
    for (int d1 = -1; d1 <= 1; ++d1)
        for (int d2 = lo2; d2 <= hi2; ++d2)
            for (int d3 = lo3; d3 <= hi3; ++d3) {
                int nz = (d1 != 0) + (d2 != 0) + (d3 != 0);
                if (!o_in_neigh(kind, nz)) continue;
                s->off[s->n][0] = d1; s->off[s->n][1] = d2; s->off[s->n][2] = d3;
                s->w[s->n] = o_default_weight(kind, nz);
                s->n++;
            }
    }
    if (coeffs) {
        if (ncoeffs != s->n && ncoeffs != s->n + 1) return -1;
        for (int j = 0; j < s->n; ++j) s->w[j] = coeffs[j];
        if (ncoeffs == s->n + 1 && coeffs[s->n] != 0.0f) { s->has_c = 1; s->c = coeffs[s->n]; }
    }
    return 0;
}

/* Eq. 1 at one point, canonical order (R4):
 *   plain: acc = w0*x0; acc = acc + wj*xj  (two roundings per term)
 *   fused: acc = w0*x0; acc = fmaf(wj, xj, acc)
 *   then acc = acc + c when c != 0. */
static float o_point_linear(const o_stencil* s, const float* src, int64_t idx,
                            const int64_t* stride, int mode) {
    float acc = s->w[0] * src[idx + s->off[0][0] * stride[0] + s->off[0][1] * stride[1]
                                  + s->off[0][2] * stride[2]];
    for (int j = 1; j < s->n; ++j) {
        float x = src[idx + s->off[j][0] * stride[0] + s->off[j][1] * stride[1]
                          + s->off[j][2] * stride[2]];
        if (mode == O_MODE_FUSED) acc = fmaf(s->w[j], x, acc);
        else { float p = s->w[j] * x; acc = acc + p; }
    }
    if (s->has_c) acc = acc + s->c;
    return acc;
}

/* Gradient-2D (reading R1, gradient-magnitude-normalised diffusion):
 *   gx = 0.5(e-w), gy = 0.5(s-n), g2 = (1+gx^2)+gy^2,
 *   lap = ((n-c)+(s-c))+((e-c)+(w-c)),  out = c + (kappa*lap)/sqrt(g2). */
static float o_point_gradient(const o_stencil* s, const float* src, int64_t idx,
                              int64_t sx, int mode) {
    float n = src[idx - sx], so = src[idx + sx];
    float w = src[idx - 1], e = src[idx + 1], c = src[idx];
    float gx = 0.5f * (e - w);
    float gy = 0.5f * (so - n);
    float g2;
    if (mode == O_MODE_FUSED) g2 = fmaf(gy, gy, fmaf(gx, gx, 1.0f));
    else { float a = gx * gx; float b = gy * gy; g2 = (1.0f + a) + b; }
    float lap = ((n - c) + (so - c)) + ((e - c) + (w - c));
    float q = (s->kappa * lap) / sqrtf(g2);
    return c + q;
}

/* Public: naive time stepping.  dims = full extents incl. the fixed ring.
 * Returns 0, or -1 on invalid arguments. */
int oracle_run(int kind, int ndims, const int64_t* dims, const float* coeffs, int ncoeffs,
               const float* in, float* out, int64_t T, int mode, int nthreads) {
    o_stencil s;
    if (o_build(kind, coeffs, ncoeffs, &s) != 0) return -1;
    if (ndims != s.ndims || T < 0 || !in || !out) return -1;
    if (mode != O_MODE_PLAIN && mode != O_MODE_FUSED) return -1;
    int64_t S1 = dims[0], S2 = (ndims >= 2) ? dims[1] : 1, S3 = (ndims == 3) ? dims[2] : 1;
    if (S1 < 2 * o_kind_radius(kind) + 1 || (ndims >= 2 && S2 < 3) || (ndims == 3 && S3 < 3)) return -1;
    int64_t n = S1 * S2 * S3;
    int64_t stride[3] = { S2 * S3, S3, 1 };
    if (ndims == 2) { stride[0] = S2; stride[1] = 1; stride[2] = 0; }
    if (ndims == 1) { stride[0] = 1; stride[1] = 0; stride[2] = 0; }
    float* plane[2];
    plane[0] = out;
    plane[1] = (float*)malloc((size_t)n * sizeof(float));
    if (!plane[1]) return -3;
    memcpy(plane[0], in, (size_t)n * sizeof(float));
    memcpy(plane[1], in, (size_t)n * sizeof(float));   /* ring in both planes */
    int nt = nthreads > 0 ? nthreads : omp_get_max_threads();
    for (int64_t t = 1; t <= T; ++t) {
        const float* src = plane[(t - 1) & 1];
        float* dst = plane[t & 1];
        if (ndims == 1) {
            /* the fixed ring is r cells wide for a radius-r neighbourhood (reading R2) */
            const int64_t r = o_kind_radius(kind);
            #pragma omp parallel for num_threads(nt) schedule(static)
            for (int64_t x = r; x < S1 - r; ++x) dst[x] = o_point_linear(&s, src, x, stride, mode);
        } else if (ndims == 2) {
            #pragma omp parallel for num_threads(nt) schedule(static)
            for (int64_t x = 1; x < S1 - 1; ++x)
                for (int64_t y = 1; y < S2 - 1; ++y) {
                    int64_t idx = x * S2 + y;
                    dst[idx] = s.gradient ? o_point_gradient(&s, src, idx, S2, mode)
                                          : o_point_linear(&s, src, idx, stride, mode);
                }
        } else {
            #pragma omp parallel for num_threads(nt) schedule(static)
            for (int64_t x = 1; x < S1 - 1; ++x)
                for (int64_t y = 1; y < S2 - 1; ++y)
                    for (int64_t z = 1; z < S3 - 1; ++z) {
                        int64_t idx = (x * S2 + y) * S3 + z;
                        dst[idx] = o_point_linear(&s, src, idx, stride, mode);
                    }
        }
    }
    if (T & 1) memcpy(out, plane[1], (size_t)n * sizeof(float));
    free(plane[1]);
    return 0;
}

/* Public: the neighbourhood and default weights the oracle uses, so tests can
 * build independent checks (dense iteration matrix, Fourier symbol). */
int oracle_stencil_info(int kind, int* npts, int* offsets /* 27*3 */, float* weights /* 27 */) {
    o_stencil s;
    if (o_build(kind, NULL, 0, &s) != 0) return -1;
    *npts = s.gradient ? 5 : s.n;
    if (s.gradient) {
        int g[5][3] = { {-1, 0, 0}, {0, -1, 0}, {0, 0, 0}, {0, 1, 0}, {1, 0, 0} };
        for (int j = 0; j < 5; ++j) { for (int d = 0; d < 3; ++d) offsets[3 * j + d] = g[j][d];
                                      weights[j] = 0.0f; }
        weights[0] = s.kappa;
        return 0;
    }
    for (int j = 0; j < s.n; ++j) {
        for (int d = 0; d < 3; ++d) offsets[3 * j + d] = s.off[j][d];
        weights[j] = s.w[j];
    }
    return 0;
}

int oracle_max_threads(void) { return omp_get_max_threads(); }
