// hhc_internal.h -- host/device structures shared by the library's own .cu/.cpp
// files (never by the oracle).  See DESIGN.md §Kernels for the layouts.
#pragma once
#include <stdint.h>
#include <algorithm>
#include <vector>

#include "../../include/hhc.h"

namespace hhc {

constexpr int kCols3D = 4;          // B: 3D kernel (one float4)
constexpr int kMaxPts = 27;

// Kernel parameters for one launch = one row of hexagons.
struct HexParams {
    const float* in;        // A_0 (ring values are read from here)
    float* plane[2];        // plane[t & 1] holds level t (two-plane storage, reading R3)
    int64_t S1, S2, S3;     // full extents (S3 = 1 in 2D)
    int64_t T;
    int tT, tS1, tS2, tS3;
    int G;                  // x-groups of threads (threads = column threads * G)
    int P;                  // pitch 2 tS1 + tT (Eq. 5)
    int64_t t0;             // level of tau = 0 of this row: 1 + m tT/2
    int64_t xbase;          // x0 of hexagon 0 of this row (reading G2)
    int tau_lo, tau_hi;     // levels of the row clipped to [1, T]
    int n2, n3;             // sub-tiles along S2 (and S3 in 3D)
    int J;                  // 3D: thread blocks per hexagonal slab (pipelined along S2)
    unsigned* flags;        // 3D, J > 1: progress flags [w][n2]
    unsigned epoch;         // flag value base for this row
    float* faceg;           // 2D, J > 1: face scratch [w][n2][tT][NX][2]
    float w[kMaxPts];       // weights in canonical order (reading R4)
    float c;                // Eq. 1 constant
    float kappa;            // Gradient-2D
    int compute_only;       // K4: skip all global<->shared transfers (Citer micro-benchmark)
    int R;                  // stencil radius = fixed-ring width (1; 2-4 for the f4 kinds, 1D)
    // f1, non-redundant hexagon-aligned multi-GPU (2D): the neighbour ranks' planes
    // (indexed by global x like plane[]) and the global rows [peer_lo, peer_hi) each
    // stores; K1 writes facet rows in those ranges into them too (peer stores)
    int npeer;
    float* peer[2][2];      // [side: lower x, upper x][parity]
    int64_t peer_lo[2], peer_hi[2];
};

// Radius of a kind's neighbourhood (1D binomial smoothers of radius 2-4).
inline int kind_radius(int kind) {
    return kind == STENCIL_BINOM1D_R2 ? 2 : kind == STENCIL_BINOM1D_R3 ? 3 : kind == STENCIL_BINOM1D_R4 ? 4 : 1;
}

// Shared-memory bytes of the HHC kernels (DESIGN.md §Kernels K1/K2): two parity
// planes in skewed coordinates, a double-buffered skewed face and the
// per-level footprint geometry table.
inline int64_t smem_bytes(int ndims, int tT, int tS1, int tS2, int tS3, int R = 1) {
    const int64_t NX = tS1 + tT + 2;
    const int64_t geo = 16 * (int64_t)tT;              // per-level geometry table (ints)
    if (ndims == 1) {
        // K0: two planes of NX1 = tS1 + R tT + 2R values, each with 4 guard floats in
        // front and >= 8 behind (aligned 4-chunk windows), + the geometry table
        const int64_t NX1 = tS1 + (int64_t)R * tT + 2 * R;
        return 4 * (2 * (((NX1 + 8 + 3) & ~3) + 4) + geo);
    }
    if (ndims == 2) return 4 * ((2 * NX + 1) * (tS2 + 8) + 2 * (int64_t)tT * NX * 2 + geo + NX + 2 * (int64_t)tT + 2 + 2 * NX);
    return 4 * (2 * NX * (tS2 + 2) * (tS3 + 4) + 2 * (int64_t)tT * NX * (tS2 + 2) * 2 + geo);
}

// Column threads of one x-group: 2D K1 threads own 8 columns (4 pairs of the
// pair layout), 3D K2 threads 4 consecutive tS3 columns of one tS2 line.
// Largest block the HHC kernels launch with (their __launch_bounds__).
// kind = 0: the largest over the kinds of that dimension (the model's bound).
inline int max_block_threads(int ndims, int kind = 0) {
    return ndims == 1 ? 256 : ndims == 2 ? ((kind == 0 || kind == STENCIL_GRADIENT2D) ? 512 : 384) : 512;
}

inline int column_threads(int ndims, int tS2, int tS3) {
    return ndims == 1 ? 256 : ndims == 2 ? tS2 / 8 : (tS3 / kCols3D) * tS2;
}

typedef void (*hex_kernel_t)(HexParams);
hex_kernel_t get_hex_kernel(int ndims, int kind, int mode, bool has_c, bool defw, int s2, int s3 = 0);
int hex_kernel_regs(int ndims, int kind, int mode, bool has_c, bool defw, int s2, int s3 = 0);
void launch_copy_ring(const float* in, float* out, int64_t S1, int64_t S2, int64_t S3, void* stream, int R = 1);
void launch_copy_full(const float* in, float* out, int64_t n, void* stream);

void set_compute_only(stencil_t h, int on);
void set_last_launches(stencil_t h, int64_t n);
int handle_radius(stencil_t h);
void handle_info(stencil_t h, int* kind, int* ndims, int64_t* dims, int* device);
int handle_clone(stencil_t h, const int64_t* dims, int maxJ, stencil_t* out);

// ---- wavefront-parallel Jacobi-1D (reading W1)
// Parallelogram tiles in skewed coordinates x' = x + t: tile (i, j) computes the
// levels t in (i*tT, min((i+1)*tT, T)] at x' in [j*tS, (j+1)*tS).  Wavefront d
// holds the tiles with i + j = d that contain an interior point; they are
// independent (one launch per wavefront) and form a contiguous i range.
struct WaveLaunch {
    int64_t d, ia, n;      // tiles i = ia .. ia+n-1, j = d - i
    int nlev_max;          // levels of the tallest tile of the wavefront
};
inline void wave1d_schedule(int64_t S, int64_t T, int tT, int tS, std::vector<WaveLaunch>& out) {
    out.clear();
    const int64_t n = S - 2, Nt = (T + tT - 1) / tT;
    if (n <= 0 || T <= 0) return;
    auto jlo = [&](int64_t i) { return (1 + i * tT + 1) / tS; };
    auto jhi = [&](int64_t i) { return (n + std::min<int64_t>((i + 1) * tT, T)) / tS; };
    const int64_t dmin = jlo(0), dmax = Nt - 1 + jhi(Nt - 1);
    int64_t ia = 0, ib = -1;
    for (int64_t d = dmin; d <= dmax; ++d) {
        while (ia < Nt && ia + jhi(ia) < d) ++ia;             // suffix: i + jhi(i) >= d
        while (ib + 1 < Nt && ib + 1 + jlo(ib + 1) <= d) ++ib;  // prefix: i + jlo(i) <= d
        if (ia > ib) continue;
        const int64_t last = std::min<int64_t>(tT, T - ib * tT);
        out.push_back(WaveLaunch{d, ia, ib - ia + 1, ib > ia ? tT : (int)last});
    }
}
// two level rows of tS + 2 slots, each padded to 16 B with slot 2 aligned, + the halo table
inline int64_t wave1d_smem_bytes(int tT, int tS) { return 4 * (2 * (((int64_t)tS + 4 + 3) & ~3) + 2 * (int64_t)tT); }

struct WaveParams {
    float* plane[2];       // plane[t & 1] holds level t (ring in both)
    int64_t S, T, d, ia;
    int tT, tS;
    float w[3], c;
};
int launch_wave1d(int mode, bool has_c, bool defw, const WaveParams& p, int64_t nblocks, void* stream);
int prepare_wave1d(int mode, bool has_c, bool defw, int tT, int tS);

// Microbenchmarks (microbench.cu)
int run_microbench(int which, int kind, int ndims, const int64_t* dims, int64_t T,
                   stencil_tile tile, int threads, double* value);

}  // namespace hhc
