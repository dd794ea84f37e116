// model.cpp -- the paper's analytical execution-time model (§4,
// Eqs. 2-30) and the tile-size optimisation of §6.1 (Eq. 31,
// P:L1365-1453), host fp64.  Two geometries (reading M1):
//   PAPER -- the printed equations (readings M2-M5 for the garbled ones);
//   EXACT -- the same equations on the hexagon and footprints the kernels
//            implement (readings G1-G3), with Eq. 2's per-row sum.
// Multi-GPU term (n_gpus > 1): DESIGN.md reading M7.
#include <algorithm>
#include <cmath>
#include <cstdint>
#include <limits>
#include <vector>

#include "hhc_internal.h"

namespace {

inline int64_t cdiv(int64_t a, int64_t b) { return (a + b - 1) / b; }

// Stencil radius of the kind being modelled (1; 2-4 for the f4 kinds, reading F4:
// slopes, pitch, footprints and facets scale by R), set by model_predict.
thread_local int64_t g_R = 1;
// Reading M8 for 2D: set while M7 evaluates a slab sub-problem -- the library runs
// those in planes mode, where a 2D hexagonal prism is split over J pipelined blocks.
thread_local bool g_planes = false;

int ndims_of(int kind) {
    switch (kind) {
    case STENCIL_JACOBI2D_5PT: case STENCIL_HEAT2D_9PT: case STENCIL_GRADIENT2D:
    case STENCIL_LAPLACIAN2D_5PT: return 2;
    case STENCIL_HEAT3D_7PT: case STENCIL_LAPLACIAN3D_27PT: return 3;
    case STENCIL_JACOBI1D_3PT: case STENCIL_BINOM1D_R2: case STENCIL_BINOM1D_R3: case STENCIL_BINOM1D_R4: return 1;
    default: return 0;
    }
}

bool tile_ok(int nd, const stencil_tile& t) {
    if (nd == 1) return t.t >= 2 && !(t.t & 1) && t.s1 >= 1;
    if (t.t < 2 || (t.t & 1) || t.s1 < 1 || t.s2 < 1) return false;
    if (nd == 2) return t.s2 % 32 == 0;
    return t.s3 >= 32 && t.s3 % 32 == 0;
}

// ---------------------------------------------------------------- PAPER
// Jacobi-1D, Section 4.1 as printed: Eqs. 3-9, Ttile by Eq. 10 (k = 1) or Eq. 12
// (k > 1), Talg by Eq. 6.
double talg_paper_1d(const int64_t* S, int64_t T, const stencil_tile& tl, const model_hw_params& hw) {
    const int64_t tT = tl.t, tS = tl.s1, S1 = S[0];
    const int64_t r = T - (T / tT) * tT;
    const int64_t Nw = 2 * cdiv(T, tT) + ((r > 0 && 2 * r <= tT) ? 0 : 1);      // Eq. 3
    const int64_t R = g_R;                                                      // reading F4 (f4 kinds)
    const int64_t wtile = tS + R * (tT - 2);                                    // Eq. 4
    const int64_t w = cdiv(S1, 2 * tS + R * tT);                                // Eq. 5
    const double m_prime = 2.0 * (double)(tS + 2 * R * tT) * hw.L_s_per_word + 2.0 * hw.tau_sync_s;   // Eqs. 7-8
    double sum = 0.0;
    for (int64_t x = tS; x <= wtile; x += 2 * R) sum += (double)cdiv(x, hw.n_v);
    const double c = 2.0 * hw.C_iter_s * sum + (double)tT * hw.tau_sync_s;       // Eq. 9
    const int64_t Mbytes = 4 * 2 * (wtile + 2 * R);                              // Mtile = 2(wtile + 2R)
    if (Mbytes > hw.m_block_bytes) return std::numeric_limits<double>::infinity();
    const int64_t k = std::min<int64_t>(hw.m_sm_bytes / Mbytes, hw.mtb_sm);     // Eq. 11 (reading M4)
    if (k < 1) return std::numeric_limits<double>::infinity();
    const double Ttile = k == 1 ? m_prime + c : m_prime + c + (double)(k - 1) * std::max(m_prime, c);   // Eq. 10/12
    return (double)Nw * Ttile * (double)cdiv(cdiv(w, k), hw.n_sm) + (double)Nw * hw.T_sync_s;        // Eq. 6
}

double talg_paper(int nd, const int64_t* S, int64_t T, const stencil_tile& tl, const model_hw_params& hw) {
    if (nd == 1) return talg_paper_1d(S, T, tl, hw);
    const int64_t tT = tl.t, tS1 = tl.s1, tS2 = tl.s2, tS3 = nd == 3 ? tl.s3 : 1;
    const int64_t S1 = S[0], S2 = S[1], S3 = nd == 3 ? S[2] : 1;
    // Eq. 3: Nw = 2 ceil(T/tT) + eps, eps = 0 iff 0 < T - floor(T/tT) tT <= tT/2
    const int64_t r = T - (T / tT) * tT;
    const int64_t Nw = 2 * cdiv(T, tT) + ((r > 0 && 2 * r <= tT) ? 0 : 1);
    const int64_t wtile = tS1 + tT - 2;                        // Eq. 4 / 21
    const int64_t w = cdiv(S1, 2 * tS1 + tT);                 // Eq. 5 / 22 (reading M2)
    const int64_t inner = nd == 2 ? tS2 : tS2 * tS3;
    const double mi = (double)inner * (double)(tS1 + 2 * tT);  // Eq. 13 / 24
    const double mo = mi;
    const double m_prime = (mi + mo) * hw.L_s_per_word + 2.0 * hw.tau_sync_s;   // Eq. 14 / 25
    double sum = 0.0;                                          // Eq. 15 / 27
    for (int64_t x = tS1; x <= wtile; x += 2) sum += (double)cdiv(x * inner, hw.n_v);
    const double c = 2.0 * hw.C_iter_s * sum + (double)tT * hw.tau_sync_s;
    int64_t Mtile;                                             // Eq. 19, reading M3 in 3D (words)
    double Nsub;
    if (nd == 2) {
        Mtile = 2 * (tS1 + tT + 1) * (tS2 + tT + 1);
        Nsub = (double)cdiv(S2 + tT, tS2);                     // Eq. 16
    } else {
        Mtile = 2 * (tS1 + tT + 1) * (tS2 + tT + 1) * (tS3 + tT + 1);
        Nsub = std::ceil(((double)(S2 + tT) / (double)tS2) * ((double)(S3 + tT) / (double)tS3));   // Eq. 23
    }
    const int64_t Mbytes = 4 * Mtile;
    if (Mbytes > hw.m_block_bytes) return std::numeric_limits<double>::infinity();   // Eq. 31
    int64_t k = std::min<int64_t>(hw.m_sm_bytes / Mbytes, hw.mtb_sm);               // Eq. 11 (reading M4)
    if (k < 1) return std::numeric_limits<double>::infinity();
    double Tprism;
    if (k == 1) Tprism = (m_prime + c) * Nsub;                                     // Eq. 16 / 28
    else Tprism = m_prime + (double)k * std::max(m_prime, c) * Nsub;               // Eq. 16 / 29
    const double rounds = (double)cdiv(cdiv(w, k), hw.n_sm);
    return (double)Nw * hw.T_sync_s + (double)Nw * Tprism * rounds;                // Eq. 17 / 30
}

// ---------------------------------------------------------------- EXACT
inline int64_t row_width(int64_t tau, int64_t tS1, int64_t tT) { return tS1 + 2 * g_R * std::min(tau, tT - tau); }

int default_threads(int nd, const stencil_tile& t) {
    const int base = hhc::column_threads(nd, t.s2, t.s3);
    const int G = base <= 256 ? std::max(1, std::min(4, 256 / base)) : 1;
    return base * G;
}

// Eq. 11's k under the CUDA occupancy rules (reading M4): shared memory per block
// plus the 1 KB the driver reserves per block, registers allocated per warp in
// units of 256 from one of the 4 sub-partition register files (RSM/4 each), at
// most MTBSM blocks and max_threads_sm threads per SM.
int64_t k_exact(int64_t Mtile, int64_t threads, const model_hw_params& hw) {
    const int64_t maxthr = hw.max_threads_sm > 0 ? hw.max_threads_sm : 2048;
    int64_t k = std::min<int64_t>({hw.m_sm_bytes / (Mtile + 1024), (int64_t)hw.mtb_sm, maxthr / threads});
    if (hw.regs_per_thread > 0) {
        const int64_t per_warp = cdiv(32 * (int64_t)hw.regs_per_thread, 256) * 256;
        k = std::min<int64_t>(k, 4 * ((hw.r_sm / 4) / per_warp) / cdiv(threads, 32));
    }
    return k;
}

double talg_exact(int nd, const int64_t* S, int64_t T, const stencil_tile& tl, const model_hw_params& hw) {
    const int64_t tT = tl.t, tS1 = tl.s1, tS2 = tl.s2, tS3 = nd == 3 ? tl.s3 : 1;
    const int64_t S1 = S[0], S2 = S[1], S3 = nd == 3 ? S[2] : 1;
    const int64_t R = g_R;
    const int64_t Mtile = hhc::smem_bytes(nd, (int)tT, (int)tS1, (int)tS2, (int)tS3, (int)R);
    const int threads = hw.threads > 0 ? hw.threads : default_threads(nd, tl);
    if (Mtile > hw.m_block_bytes || threads > hhc::max_block_threads(nd)) return std::numeric_limits<double>::infinity();
    const int64_t k = k_exact(Mtile, threads, hw);                                       // Eq. 11
    if (k < 1) return std::numeric_limits<double>::infinity();
    const int64_t G = nd == 1 ? 1 : std::max<int64_t>(1, threads / hhc::column_threads(nd, (int)tS2, (int)tS3));
    const int64_t P = 2 * tS1 + R * tT, h = tT / 2;
    const int64_t wA = cdiv(S1 + R * h, P);                    // reading G2 (F4: radius R)
    const int64_t wB = S1 > tS1 ? cdiv(S1 - tS1, P) : 0;
    const double L_sm = hw.L_s_per_word * hw.n_sm;             // reading M5
    const int64_t Nw = cdiv(2 * T, tT) + 1;
    double total = 0.0;
    // rows with identical (phase, lo, hi, final-level) cost the same: memoise
    int64_t key_prev[2] = {-1, -1};
    double val_prev[2] = {0.0, 0.0};
    for (int64_t m = -1; m <= Nw - 2; ++m) {
        const int64_t t0 = 1 + m * h;
        const int64_t lo = std::max<int64_t>(0, 1 - t0);
        const int64_t hi = std::min<int64_t>(tT, T - t0 + 1);
        const int64_t nlev = hi - lo;
        const int ph = (int)(((m % 2) + 2) % 2);
        const int64_t w = ph == 0 ? wA : wB;
        total += hw.T_sync_s;
        if (w == 0 || nlev <= 0) continue;
        const int64_t fin = (t0 + hi - 1 == T) ? hi - 1 : -1;
        const int64_t key = ((lo * 4096 + hi) * 4096 + (fin + 1));
        if (key == key_prev[ph]) { total += val_prev[ph]; continue; }
        // footprint (reads) and facets (writes) per unit inner extent, reading G3
        int64_t reads = 0, writes = 0, area = 0;
        double csum = 0.0;
        const int64_t inner = nd == 1 ? 1 : nd == 2 ? tS2 : tS2 * tS3;
        for (int64_t tau = lo; tau < hi; ++tau) {
            const int64_t W = row_width(tau, tS1, tT);
            area += W;
            if (tau == lo) reads += W + 2 * R;
            else if (tau <= h) reads += 4 * R;
            if (t0 + tau == T || tau == hi - 1) writes += W;
            else if (tau + 1 > h) writes += 4 * R;
            // reading M9 (geometry 2): the G x-groups split the row, so a level lasts
            // G*ceil(W/G) rows' worth of the block's vector units
            const int64_t We = (hw.geometry >= 2 && G > 1) ? G * cdiv(W, G) : W;
            csum += (double)cdiv(We * inner, hw.n_v);          // Eq. 15 / 27, row by row
            // reading M10 (geometry 3): each x-group's register window first loads the
            // rows below and at its segment -- window_rows row equivalents per group
            if (hw.geometry == 3 && nd >= 2) csum += hw.window_rows * (double)(G * inner) / (double)hw.n_v;
        }
        double Nsub, mi, mo, extra = 0.0;
        int64_t J = 1;
        if (nd == 1) {
            Nsub = 1.0;
            mi = (double)reads;
            mo = (double)writes;
        } else if (nd == 2) {
            const int64_t n2 = cdiv(S2 + nlev - 1, tS2);
            Nsub = (double)n2;
            if (g_planes) {
                // M8 in 2D (slab sub-problems): J blocks per prism, the face (2 columns per
                // row and level) written and read back through global memory
                J = std::max<int64_t>(1, std::min<int64_t>(n2, ((int64_t)hw.n_sm * k) / w));
                if (J > 1) {
                    Nsub = (double)(cdiv(n2, J) + (J - 1));
                    extra = 4.0 * (double)area;
                }
            }
            mi = (double)reads * (double)(tS2 + 2);
            mo = (double)writes * (double)tS2;
        } else {
            // reading M8: J blocks per slab pipelined along S2 (the library's choice);
            // a block sweeps ceil(n2/J)*n3 sub-slabs, the last starts J-1 sub-slabs late
            const int64_t n2 = cdiv(S2 + nlev - 1, tS2), n3 = cdiv(S3 + nlev - 1, tS3);
            J = std::max<int64_t>(1, std::min<int64_t>(n2, ((int64_t)hw.n_sm * k) / w));
            Nsub = (double)(cdiv(n2, J) * n3 + (J - 1));
            mi = (double)reads * (double)((tS2 + 2) * (tS3 + 2));
            mo = (double)writes * (double)(tS2 * tS3);
            extra = 4.0 * (double)tS3 * (double)area;           // S2 face through global memory
        }
        const double m_prime = (mi + mo + extra) * L_sm + 2.0 * hw.tau_sync_s;     // Eq. 14 / 25
        const double c = csum * hw.C_iter_s + (double)nlev * hw.tau_sync_s;
        double Tprism;
        if (k == 1) Tprism = (m_prime + c) * Nsub;                                 // Eq. 16 / 28
        else Tprism = m_prime + (double)k * std::max(m_prime, c) * Nsub;           // Eq. 16 / 29
        const double v = Tprism * (double)cdiv(cdiv(w * J, k), hw.n_sm);          // Eq. 2
        key_prev[ph] = key;
        val_prev[ph] = v;
        total += v;
    }
    return total;
}

// Reading M7 (multi-GPU, not in the paper; BASELINE.json north_star): G slabs of
// own = ceil(S1/G) interior rows along S1, ghost depth g = tT, time tiles of
// Tt = tT steps (the last one T - (n-1) tT).  The busiest rank has e = 2
// neighbours (e = 1 when G = 2).  Per tile, with T_exch = g * plane * 4 B / link
// bandwidth + latency:
//   plain   (dist_overlap = 0): Talg(own + e g, Tt) + T_exch
//   overlap (dist_overlap = 1): Talg(own, Tt) + e Talg(3 g, Tt) + max(0, T_exch - Talg(own, Tt))
// (the edge sub-slabs of 3g rows run besides the ghost-free interior, which hides
// the exchange).  T_G = the sum over the tiles.
double talg_dist(int nd, const int64_t* S, int64_t T, const stencil_tile& tl, const model_hw_params& hw,
                 double (*f)(int, const int64_t*, int64_t, const stencil_tile&, const model_hw_params&)) {
    const int64_t G = hw.n_gpus;
    const int64_t g = tl.t;
    const int64_t own = cdiv(S[0], G);
    const int64_t e = G >= 3 ? 2 : 1;
    const double plane = (double)S[1] * (double)(nd == 3 ? S[2] : 1) * 4.0;
    const double bw = hw.link_bytes_per_s > 0 ? hw.link_bytes_per_s : 7.7e11;
    const double t_exch = (double)g * plane / bw + hw.link_latency_s;
    auto run = [&](int64_t rows, int64_t Tt) {
        const int64_t Sl[3] = {rows, S[1], nd == 3 ? S[2] : 1};
        g_planes = true;
        const double v = f(nd, Sl, Tt, tl, hw);
        g_planes = false;
        return v;
    };
    const int64_t n = cdiv(T, tl.t);
    const int64_t Tlast = T - (n - 1) * tl.t;
    double total = 0.0;
    for (int pass = 0; pass < 2; ++pass) {            // pass 0: the n-1 full tiles, pass 1: the last one
        const int64_t Tt = pass == 0 ? tl.t : Tlast;
        const int64_t cnt = pass == 0 ? n - 1 : 1;
        if (cnt == 0) continue;
        double tt;
        if (hw.dist_overlap && own >= 2 * g) {
            const double ti = run(own, Tt);
            tt = ti + (double)e * run(3 * g, Tt) + std::max(0.0, t_exch - ti);
        } else {
            tt = run(own + e * g, Tt) + t_exch;
        }
        if (!std::isfinite(tt)) return tt;
        total += (double)cnt * tt;
    }
    return total;
}

}  // namespace

extern "C" double model_predict(stencil_kind kind, int ndims, const int64_t* dims, int64_t T, stencil_tile tile,
                                const model_hw_params* hw) {
    const double nan = std::numeric_limits<double>::quiet_NaN();
    if (!hw || !dims || ndims != ndims_of(kind) || T < 1) return nan;
    for (int d = 0; d < ndims; ++d)
        if (dims[d] < 3) return nan;
    if (!tile_ok(ndims, tile)) return nan;
    if (hw->n_sm < 1 || hw->n_v < 1 || hw->mtb_sm < 1 || hw->m_sm_bytes < 1 || hw->m_block_bytes < 1) return nan;
    const int R = hhc::kind_radius(kind);
    if (dims[0] < 2 * R + 1) return nan;
    int64_t S[3] = {dims[0] - 2 * R, ndims >= 2 ? dims[1] - 2 : 1, ndims == 3 ? dims[2] - 2 : 1};
    auto f = hw->geometry >= 1 ? talg_exact : talg_paper;
    g_R = R;
    const double v = (hw->n_gpus > 1 && R == 1) ? talg_dist(ndims, S, T, tile, *hw, f) : f(ndims, S, T, tile, *hw);
    g_R = 1;
    return v;
}

// Wavefront-parallel Jacobi-1D: "the total execution time is
// the sum of the times for each wavefront ... equation 6 holds for wavefront
// parallel codes".  Eq. 6 per wavefront d of n_d parallelogram
// tiles: T_sync + ceil(ceil(n_d/k)/nSM) * Ttile, Ttile by Eq. 10 (k = 1) or
// Eq. 12 (k > 1) with Eq. 8's m' = (mi + mo) L + 2 tau_sync and Eq. 9's
// c = sum over the tile's rows of C_iter ceil(tS/nV) + tau_sync.  Footprint of a
// tile of nlev levels (reading W1): mi = tS + 2 + 2(nlev-1) words in
// (bottom row + left halo), mo = tS + 2(nlev-1) out (top row + right edge).
extern "C" double model_predict_wavefront(stencil_kind kind, int ndims, const int64_t* dims, int64_t T,
                                          stencil_tile tile, const model_hw_params* hw) {
    const double nan = std::numeric_limits<double>::quiet_NaN();
    if (!hw || !dims || kind != STENCIL_JACOBI1D_3PT || ndims != 1 || T < 1 || dims[0] < 3) return nan;
    if (tile.t < 1 || tile.s1 < 2) return nan;
    if (hw->n_sm < 1 || hw->n_v < 1 || hw->mtb_sm < 1 || hw->m_sm_bytes < 1 || hw->m_block_bytes < 1) return nan;
    const double inf = std::numeric_limits<double>::infinity();
    const int64_t tS = tile.s1;
    const int64_t Mtile = hhc::wave1d_smem_bytes(tile.t, tile.s1);
    if (Mtile > hw->m_block_bytes) return inf;
    int64_t k = std::min<int64_t>(hw->m_sm_bytes / Mtile, hw->mtb_sm);         // Eq. 11
    if (hw->geometry == 1) k = k_exact(Mtile, 256, *hw);                        // reading M4
    if (k < 1) return inf;
    const double L = hw->geometry == 1 ? hw->L_s_per_word * hw->n_sm : hw->L_s_per_word;   // reading M5
    std::vector<hhc::WaveLaunch> ws;
    hhc::wave1d_schedule(dims[0], T, tile.t, tile.s1, ws);
    double total = 0.0;
    for (const auto& w : ws) {
        const int64_t nl = w.nlev_max;
        const double mi = (double)(tS + 2 + 2 * (nl - 1)), mo = (double)(tS + 2 * (nl - 1));
        const double m_prime = (mi + mo) * L + 2.0 * hw->tau_sync_s;                      // Eq. 8
        const double c = (double)nl * (hw->C_iter_s * (double)cdiv(tS, hw->n_v) + hw->tau_sync_s);   // Eq. 9
        if (hw->geometry == 1) {
            // reading W2: the busiest SM holds ceil(n_d / nSM) tiles (round-robin), min(k, that) at a time
            const int64_t m = cdiv(w.n, hw->n_sm), ke = std::min(k, m);
            const double Ttile = ke == 1 ? m_prime + c : m_prime + c + (double)(ke - 1) * std::max(m_prime, c);
            total += hw->T_sync_s + Ttile * (double)cdiv(m, ke);
        } else {
            const double Ttile = k == 1 ? m_prime + c : m_prime + c + (double)(k - 1) * std::max(m_prime, c);   // Eq. 10/12
            total += hw->T_sync_s + Ttile * (double)cdiv(cdiv(w.n, k), hw->n_sm);            // Eq. 6
        }
    }
    return total;
}

// The wavefront schedule's tile by exhaustive enumeration of Talg (Eq. 31's
// argmin, on model_predict_wavefront; reading W3):
// tT in [1, min(T, 128)], tS in {4, 6, 8, 12, 16, ..., 2^k, 1.5 * 2^k, ...} up to
// min(16384, the 4-rounded S + T); ties -> the smallest (t, s1).
extern "C" int model_select_wavefront_tile(stencil_kind kind, int ndims, const int64_t* dims, int64_t T,
                                           const model_hw_params* hw, double within, stencil_tile* best,
                                           stencil_tile* cands, int cap, int* n_cands) {
    if (!hw || !dims || !best || kind != STENCIL_JACOBI1D_3PT || ndims != 1 || T < 1 || dims[0] < 3 || within < 0)
        return STENCIL_EINVAL;
    std::vector<int> tss;
    const int64_t smax = std::min<int64_t>(16384, ((dims[0] - 2 + T) + 3) / 4 * 4);
    for (int64_t p = 4; p <= smax; p *= 2) {
        tss.push_back((int)p);
        if (p * 3 / 2 <= smax && p >= 4) tss.push_back((int)(p * 3 / 2));
    }
    std::sort(tss.begin(), tss.end());
    tss.erase(std::unique(tss.begin(), tss.end()), tss.end());
    std::vector<std::pair<stencil_tile, double>> vals;
    double bt = std::numeric_limits<double>::infinity();
    stencil_tile bb{0, 0, 0, 0};
    for (int t = 1; t <= std::min<int64_t>(T, 128); ++t)
        for (int ts : tss) {
            stencil_tile tl{t, ts, 0, 0};
            const double v = model_predict_wavefront(kind, 1, dims, T, tl, hw);
            if (!std::isfinite(v)) continue;
            vals.push_back({tl, v});
            if (v < bt) { bt = v; bb = tl; }
        }
    if (!std::isfinite(bt)) return STENCIL_ETILE;
    *best = bb;
    int n = 0;
    for (auto& e : vals)
        if (e.second <= (1.0 + within) * bt) {
            if (cands && n < cap) cands[n] = e.first;
            ++n;
        }
    if (n_cands) *n_cands = n;
    return STENCIL_OK;
}

extern "C" int model_select_tile(stencil_kind kind, int ndims, const int64_t* dims, int64_t T,
                                 const model_hw_params* hw, double within, stencil_tile* best, int* best_threads,
                                 stencil_tile* cands, int cap, int* n_cands) {
    if (!hw || !dims || !best || ndims != ndims_of(kind) || T < 1 || within < 0) return STENCIL_EINVAL;
    for (int d = 0; d < ndims; ++d)
        if (dims[d] < 3) return STENCIL_EINVAL;
    // search space, reading M6
    const int64_t S1 = dims[0] - 2 * hhc::kind_radius(kind), S2 = ndims >= 2 ? dims[1] - 2 : 1,
                  S3 = ndims == 3 ? dims[2] - 2 : 1;
    if (S1 < 1) return STENCIL_EINVAL;
    const int64_t Tev = T + (T & 1);
    const int64_t tTmax = std::min<int64_t>(Tev, 128), tS1max = std::min<int64_t>(S1, 64);
    const int64_t innerS = ndims == 2 ? S2 : S3;
    const int64_t innermax = std::min<int64_t>(1024, cdiv(innerS, 32) * 32);
    const int64_t tS2max3 = std::min<int64_t>(S2, 16);
    struct V { stencil_tile t; double v; };
    std::vector<V> vals;
    stencil_tile bt{0, 0, 0, 0};
    double bv = std::numeric_limits<double>::infinity();
    if (ndims == 1) {
        // reading M6 (1D): tS1 in 32..min(S1 rounded up to 32, 4096) step 32
        const int64_t lim = std::min<int64_t>(cdiv(S1, 32) * 32, 4096);
        for (int64_t tT = 2; tT <= tTmax; tT += 2)
            for (int64_t tS1 = 32; tS1 <= lim; tS1 += 32) {
                const stencil_tile t{(int)tT, (int)tS1, 0, 0};
                const double v = model_predict(kind, ndims, dims, T, t, hw);
                if (!std::isfinite(v)) continue;
                vals.push_back(V{t, v});
                if (v < bv) { bv = v; bt = t; }
            }
    }
    for (int64_t tT = 2; ndims > 1 && tT <= tTmax; tT += 2)
        for (int64_t tS1 = 1; tS1 <= tS1max; ++tS1) {
            const int64_t n2 = ndims == 2 ? 1 : tS2max3;
            for (int64_t a = 1; a <= n2; ++a)
                for (int64_t in = 32; in <= innermax; in += 32) {
                    stencil_tile t;
                    t.t = (int)tT; t.s1 = (int)tS1;
                    if (ndims == 2) { t.s2 = (int)in; t.s3 = 0; }
                    else { t.s2 = (int)a; t.s3 = (int)in; }
                    const double v = model_predict(kind, ndims, dims, T, t, hw);
                    if (!std::isfinite(v)) {
                        if (ndims == 2 || true) {
                            // larger inner tiles only grow Mtile: stop this inner sweep
                            if (std::isinf(v)) break;
                        }
                        continue;
                    }
                    vals.push_back(V{t, v});
                    if (v < bv) { bv = v; bt = t; }   // strict: first (lexicographic) minimum wins
                }
        }
    if (!std::isfinite(bv)) return STENCIL_ETILE;
    *best = bt;
    if (best_threads) *best_threads = default_threads(ndims, bt);
    int n = 0;
    for (auto& x : vals)
        if (x.v <= (1.0 + within) * bv) {
            if (cands && n < cap) cands[n] = x.t;
            ++n;
        }
    if (n_cands) *n_cands = n;
    return STENCIL_OK;
}
