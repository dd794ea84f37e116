// hhc_api.cu -- the C ABI of include/hhc.h: handles, planning (§8(a) a1-a3),
// buffer roles (a2), the row-of-hexagons launch sequence captured as a CUDA
// graph (a3), and host-buffer runs for the end-to-end measurement.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdlib>
#include <cstring>
#include <vector>

#include "hhc_internal.h"

using namespace hhc;

namespace {

int kind_ndims_host(int kind) {
    switch (kind) {
    case STENCIL_JACOBI2D_5PT: case STENCIL_HEAT2D_9PT: case STENCIL_GRADIENT2D:
    case STENCIL_LAPLACIAN2D_5PT: return 2;
    case STENCIL_HEAT3D_7PT: case STENCIL_LAPLACIAN3D_27PT: return 3;
    case STENCIL_JACOBI1D_3PT: case STENCIL_BINOM1D_R2: case STENCIL_BINOM1D_R3: case STENCIL_BINOM1D_R4: return 1;
    default: return 0;
    }
}

// Default weights (reading R1) by number of non-zero offset components.
float default_weight(int kind, int nz) {
    switch (kind) {
    case STENCIL_JACOBI2D_5PT: return 0.2f;
    case STENCIL_JACOBI1D_3PT: return 1.0f / 3.0f;
    case STENCIL_LAPLACIAN2D_5PT: return nz == 0 ? 0.5f : 0.125f;
    case STENCIL_HEAT2D_9PT: return nz == 0 ? 0.25f : (nz == 1 ? 0.125f : 0.0625f);
    case STENCIL_HEAT3D_7PT: return nz == 0 ? 0.25f : 0.125f;
    case STENCIL_LAPLACIAN3D_27PT:
        return nz == 0 ? 0.5f : nz == 1 ? 7.0f / 128.0f : nz == 2 ? 3.0f / 256.0f : 1.0f / 256.0f;
    default: return 0.0f;
    }
}

bool in_nb(int kind, int nz) {
    return (kind == STENCIL_HEAT2D_9PT || kind == STENCIL_LAPLACIAN3D_27PT || kind == STENCIL_JACOBI1D_3PT) ? true
                                                                                                           : nz <= 1;
}


struct RowPlan {
    int m;
    int64_t t0, xbase;
    int tau_lo, tau_hi;
    int w, n2, n3, J;
};

int64_t cdiv(int64_t a, int64_t b) { return (a + b - 1) / b; }

}  // namespace

struct RunSpec {
    int planes_mode;          // 0: stencil_run (in -> out); 1: stencil_run_planes
    const float* a;           // in  | plane0
    float* b;                 // out | plane1
    int64_t dims[3];
    int64_t T;
    stencil_tile tile;
    int G, thr;
};

struct GraphEntry {
    RunSpec spec;
    cudaGraphExec_t exec;
    int64_t launches;
    uint64_t last_use;
};

struct stencil_s {
    int kind = 0, ndims = 0, mode = 0;
    int64_t dims[3] = {1, 1, 1};
    int npts = 0;
    float w[kMaxPts] = {};
    float c = 0.0f, kappa = 0.125f;
    bool has_c = false;
    bool defw = true;           // default weights -> immediate-operand kernels
    int device = 0, nsm = 148, smem_optin = 227 * 1024;
    float* scratch = nullptr;
    unsigned* flags = nullptr;
    int64_t flags_n = 0;
    float* faceg = nullptr;     // 2D J > 1: face scratch [w][n2][tT][NX][2]
    int64_t faceg_n = 0;
    float* h_in_dev = nullptr;   // stencil_run_host device buffers
    float* h_out_dev = nullptr;
    float* hb_dev[2][2] = {{nullptr, nullptr}, {nullptr, nullptr}};   // stencil_run_host_batch [slot][in/out]
    cudaStream_t hb_s[2] = {nullptr, nullptr};                       // its copy streams (H2D, D2H)
    cudaEvent_t hb_ev[2][3] = {{nullptr, nullptr, nullptr}, {nullptr, nullptr, nullptr}};
    int sticky = 0;
    int64_t last_launches = 0;
    cudaStream_t cap_stream = nullptr;
    std::vector<GraphEntry> graphs;
    uint64_t use_clock = 0;
    int compute_only = 0;
    int occ = 1;
    int envJ = 0;               // HHC_J read once at create (experiments; 0 = library rule)
    int maxJ = 0;               // > 0: cap on the 3D blocks per slab (1 = never wait on flags)
    int R = 1;                  // stencil radius = fixed-ring width (f4 kinds: 2-4)

    int64_t nelem() const { return dims[0] * dims[1] * dims[2]; }
};

extern "C" const char* stencil_strerror(int status) {
    switch (status) {
    case STENCIL_OK: return "ok";
    case STENCIL_EINVAL: return "invalid argument";
    case STENCIL_ETILE: return "invalid or infeasible tile";
    case STENCIL_ENOMEM: return "out of memory";
    case STENCIL_ECUDA: return "CUDA error";
    case STENCIL_ENCCL: return "NCCL error";
    case STENCIL_ENODEV: return "no usable sm_100 device";
    default: return "unknown status";
    }
}

static void drop_graphs(stencil_t h) {
    for (auto& g : h->graphs) cudaGraphExecDestroy(g.exec);
    h->graphs.clear();
}

static int cuda_fail(stencil_t h, cudaError_t e) {
    if (e == cudaSuccess) return STENCIL_OK;
    if (h) h->sticky = STENCIL_ECUDA;
    return e == cudaErrorMemoryAllocation ? STENCIL_ENOMEM : STENCIL_ECUDA;
}

extern "C" int stencil_create(stencil_kind kind, int ndims, const int64_t* dims, const float* coeffs,
                              int ncoeffs, int mode, stencil_t* out) {
    if (!out || !dims) return STENCIL_EINVAL;
    *out = nullptr;
    const int D = kind_ndims_host(kind);
    if (D == 0 || D != ndims) return STENCIL_EINVAL;
    if (mode != STENCIL_MODE_PLAIN && mode != STENCIL_MODE_FUSED) return STENCIL_EINVAL;
    for (int d = 0; d < ndims; ++d)
        if (dims[d] < 3) return STENCIL_EINVAL;
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) return STENCIL_ENODEV;
    cudaDeviceProp prop;
    if (cudaGetDeviceProperties(&prop, dev) != cudaSuccess) return STENCIL_ENODEV;
    if (prop.major < 10) return STENCIL_ENODEV;   // sm_100a code only
    stencil_s* h = new stencil_s();
    h->kind = kind; h->ndims = ndims; h->mode = mode;
    for (int d = 0; d < ndims; ++d) h->dims[d] = dims[d];
    h->device = dev;
    h->nsm = prop.multiProcessorCount;
    h->smem_optin = (int)prop.sharedMemPerBlockOptin;
    if (kind == STENCIL_GRADIENT2D) {
        h->npts = 5;
        if (coeffs) {
            if (ncoeffs != 1) { delete h; return STENCIL_EINVAL; }
            h->kappa = coeffs[0];
            h->defw = h->kappa == 0.125f;
        }
    } else if (kind_radius(kind) > 1) {
        // f4: binomial C(2R, j) / 4^R on the offsets -R..R (reading R1)
        const int R = kind_radius(kind);
        h->R = R;
        h->npts = 2 * R + 1;
        double c = 1.0;
        for (int j = 0; j <= 2 * R; ++j) {
            h->w[j] = (float)(c / (double)(1 << (2 * R)));
            c = c * (double)(2 * R - j) / (double)(j + 1);
        }
        for (int d = 0; d < ndims; ++d)
            if (dims[d] < 2 * R + 1) { delete h; return STENCIL_EINVAL; }
        if (coeffs) {
            const int n = h->npts;
            if (ncoeffs != n && ncoeffs != n + 1) { delete h; return STENCIL_EINVAL; }
            for (int j = 0; j < n; ++j) {
                if (coeffs[j] != h->w[j] || std::signbit(coeffs[j]) != std::signbit(h->w[j])) h->defw = false;
                h->w[j] = coeffs[j];
            }
            if (ncoeffs == n + 1 && coeffs[n] != 0.0f) { h->has_c = true; h->c = coeffs[n]; h->defw = false; }
        }
    } else {
        int n = 0;
        for (int d1 = -1; d1 <= 1; ++d1)
            for (int d2 = (D >= 2 ? -1 : 0); d2 <= (D >= 2 ? 1 : 0); ++d2)
                for (int d3 = (D == 3 ? -1 : 0); d3 <= (D == 3 ? 1 : 0); ++d3) {
                    const int nz = (d1 != 0) + (d2 != 0) + (d3 != 0);
                    if (!in_nb(kind, nz)) continue;
                    h->w[n++] = default_weight(kind, nz);
                }
        h->npts = n;
        if (coeffs) {
            if (ncoeffs != n && ncoeffs != n + 1) { delete h; return STENCIL_EINVAL; }
            for (int j = 0; j < n; ++j) {
                if (coeffs[j] != h->w[j] || std::signbit(coeffs[j]) != std::signbit(h->w[j])) h->defw = false;
                h->w[j] = coeffs[j];
            }
            if (ncoeffs == n + 1 && coeffs[n] != 0.0f) { h->has_c = true; h->c = coeffs[n]; h->defw = false; }
        }
    }
    if (const char* ej = getenv("HHC_J")) h->envJ = std::max(0, atoi(ej));
    if (cudaStreamCreateWithFlags(&h->cap_stream, cudaStreamNonBlocking) != cudaSuccess) {
        delete h;
        return STENCIL_ECUDA;
    }
    *out = h;
    return STENCIL_OK;
}

extern "C" void stencil_destroy(stencil_t h) {
    if (!h) return;
    drop_graphs(h);
    if (h->scratch) cudaFree(h->scratch);
    if (h->flags) cudaFree(h->flags);
    if (h->faceg) cudaFree(h->faceg);
    if (h->h_in_dev) cudaFree(h->h_in_dev);
    if (h->h_out_dev) cudaFree(h->h_out_dev);
    for (int i = 0; i < 2; ++i) {
        for (int j = 0; j < 2; ++j)
            if (h->hb_dev[i][j]) cudaFree(h->hb_dev[i][j]);
        if (h->hb_s[i]) cudaStreamDestroy(h->hb_s[i]);
        for (int j = 0; j < 3; ++j)
            if (h->hb_ev[i][j]) cudaEventDestroy(h->hb_ev[i][j]);
    }
    if (h->cap_stream) cudaStreamDestroy(h->cap_stream);
    delete h;
}

// ---- tile validation (§8(b) validation rules; Eq. 31 integrality)
static int check_tile(int ndims, stencil_tile t, int threads, int smem_limit, int* G_out, int* thr_out,
                      int kind = 0) {
    if (t.t < 2 || (t.t & 1) || t.s1 < 1) return STENCIL_ETILE;
    if (ndims == 1) {
        if (t.t > 1024 || t.s1 > 65536) return STENCIL_ETILE;
        if (threads != 0 && threads != 256) return STENCIL_EINVAL;
        const int64_t sm = smem_bytes(1, t.t, t.s1, 0, 0, kind_radius(kind));
        if (sm > smem_limit) return STENCIL_ETILE;
        *G_out = 1;
        *thr_out = 256;
        return STENCIL_OK;
    }
    if (ndims == 2) {
        if (t.s2 < 32 || t.s2 % 32) return STENCIL_ETILE;
    } else {
        if (t.s2 < 1 || t.s3 < 32 || t.s3 % 32) return STENCIL_ETILE;
    }
    if (t.t > 1024 || t.s1 > 4096 || t.s2 > 8192 || (ndims == 3 && t.s3 > 4096)) return STENCIL_ETILE;
    const int base = column_threads(ndims, t.s2, t.s3);
    if (base > max_block_threads(ndims, kind)) return STENCIL_ETILE;
    int G;
    if (threads == 0) {
        G = base <= 256 ? std::max(1, std::min(4, 256 / base)) : 1;
    } else {
        if (threads < 0 || threads > max_block_threads(ndims, kind) || threads % base) return STENCIL_EINVAL;
        G = threads / base;
    }
    const int64_t sm = smem_bytes(ndims, t.t, t.s1, t.s2, t.s3);
    if (sm > smem_limit) return STENCIL_ETILE;
    *G_out = G;
    *thr_out = base * G;
    return STENCIL_OK;
}

extern "C" int stencil_tile_resources(stencil_kind kind, int ndims, stencil_tile tile, int threads, int mode,
                                      int64_t* smem, int* block_threads, int* regs) {
    if (ndims < 1 || ndims > 3) return STENCIL_EINVAL;
    if (kind != 0 && kind_ndims_host(kind) != ndims) return STENCIL_EINVAL;
    int G, thr;
    const int rc = check_tile(ndims, tile, threads, 227 * 1024, &G, &thr, kind);
    if (rc) return rc;
    if (smem) *smem = smem_bytes(ndims, tile.t, tile.s1, tile.s2, tile.s3, kind_radius(kind));
    if (block_threads) *block_threads = thr;
    if (regs) {
        // Eq. 11's register bound (reading M4): the kernel the library launches for this
        // (kind, mode, tile) with default weights, from cudaFuncGetAttributes; 0 if kind is 0
        // or no device is visible (the attribute query needs a CUDA context)
        *regs = kind != 0 ? hex_kernel_regs(ndims, kind, mode, false, true, tile.s2, tile.s3) : 0;
        cudaGetLastError();
    }
    return STENCIL_OK;
}

extern "C" int stencil_tile_occupancy(stencil_kind kind, int ndims, stencil_tile tile, int threads, int mode,
                                      int* blocks_per_sm) {
    if (!blocks_per_sm || kind_ndims_host(kind) != ndims) return STENCIL_EINVAL;
    int G, thr;
    const int rc = check_tile(ndims, tile, threads, 227 * 1024, &G, &thr, kind);
    if (rc) return rc;
    hex_kernel_t k = get_hex_kernel(ndims, kind, mode, false, true, tile.s2, tile.s3);
    if (!k) return STENCIL_EINVAL;
    const int64_t smem = smem_bytes(ndims, tile.t, tile.s1, tile.s2, tile.s3, kind_radius(kind));
    cudaError_t e = cudaFuncSetAttribute((const void*)k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e == cudaSuccess) e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, (const void*)k, thr, (size_t)smem);
    if (e != cudaSuccess) {
        cudaGetLastError();
        return e == cudaErrorNoDevice || e == cudaErrorInsufficientDriver ? STENCIL_ENODEV : STENCIL_ECUDA;
    }
    return STENCIL_OK;
}

// ---- planning (a1, a3): rows m = -1 .. Nw-2 (reading G2)
static void plan_rows(int ndims, const int64_t* dims, int64_t T, stencil_tile t, std::vector<RowPlan>& rows,
                      int R = 1) {
    // radius R (f4): ring of width R, interior [R, S1-1-R], rows widen by R per
    // level side, pitch P = 2 tS1 + R tT, phase B at x0 + tS1 + R tT/2
    rows.clear();
    const int64_t S1i = dims[0] - 2 * R;
    const int h = t.t / 2;
    const int P = 2 * t.s1 + R * t.t;
    const int64_t Nw = cdiv(2 * T, t.t) + 1;
    const int64_t wA = cdiv(S1i + (int64_t)R * h, P);
    const int64_t wB = S1i > t.s1 ? cdiv(S1i - t.s1, P) : 0;
    for (int64_t m = -1; m <= Nw - 2; ++m) {
        RowPlan r;
        r.m = (int)m;
        r.t0 = 1 + m * h;
        r.tau_lo = (int)std::max<int64_t>(0, 1 - r.t0);
        r.tau_hi = (int)std::min<int64_t>(t.t, T - r.t0 + 1);
        const bool A = (m % 2 == 0);
        r.xbase = A ? R : R + t.s1 + (int64_t)R * h;
        r.w = (int)(A ? wA : wB);
        const int nlev = r.tau_hi - r.tau_lo;
        if (ndims == 1) {
            r.n2 = 1;
            r.n3 = 1;
        } else if (ndims == 2) {
            r.n2 = (int)cdiv(dims[1] - 2 + nlev - 1, t.s2);
            r.n3 = 1;
        } else {
            r.n2 = (int)cdiv(dims[1] - 2 + nlev - 1, t.s2);
            r.n3 = (int)cdiv(dims[2] - 2 + nlev - 1, t.s3);
        }
        r.J = 1;
        if (nlev > 0 && r.w > 0) rows.push_back(r);
    }
}

extern "C" int stencil_plan_info(int ndims, const int64_t* dims, int64_t T, stencil_tile tile,
                                 int64_t* n_rows, int64_t* w_a, int64_t* w_b, int64_t* n_sub) {
    if (ndims < 1 || ndims > 3 || !dims || T < 1) return STENCIL_EINVAL;
    int G, thr;
    const int rc = check_tile(ndims, tile, 0, 1 << 30, &G, &thr);
    if (rc) return rc;
    std::vector<RowPlan> rows;
    plan_rows(ndims, dims, T, tile, rows);
    const int64_t S1i = dims[0] - 2;
    const int P = 2 * tile.s1 + tile.t;
    if (n_rows) *n_rows = cdiv(2 * T, tile.t) + 1;
    if (w_a) *w_a = cdiv(S1i + tile.t / 2, P);
    if (w_b) *w_b = S1i > tile.s1 ? cdiv(S1i - tile.s1, P) : 0;
    if (n_sub) {
        int64_t ns = 0;
        for (auto& r : rows) ns = std::max<int64_t>(ns, (int64_t)r.n2 * r.n3);
        *n_sub = ns;
    }
    return STENCIL_OK;
}

static int choose_J(stencil_t h, const RowPlan& r) {
    const int cap = std::max(1, h->nsm * std::max(h->occ, 1) / std::max(r.w, 1));
    int J = std::max(1, std::min(r.n2, cap));
    if (h->envJ > 0) J = std::max(1, std::min({h->envJ, r.n2, cap}));
    if (h->maxJ > 0) J = std::min(J, h->maxJ);
    return J;
}

// 2D rows get J > 1 blocks per hexagon only in planes mode (slab sub-problems of the
// multi-GPU path, where few hexagons share the GPU); full-grid runs keep J = 1.
static bool j_rows(const stencil_t h, bool planes) { return h->ndims == 3 || (h->ndims == 2 && planes); }

// Everything that must not happen inside stream capture: the kernel's smem
// attribute, its occupancy (for J), the flag buffer and the 2D face scratch.
static int prepare_rows(stencil_t h, const int64_t* dims, int64_t T, stencil_tile tile, int thr,
                        bool planes = false) {
    hex_kernel_t k = get_hex_kernel(h->ndims, h->kind, h->mode, h->has_c, h->defw, tile.s2, h->ndims == 3 ? tile.s3 : 0);
    if (!k) return STENCIL_EINVAL;
    const int64_t smem = smem_bytes(h->ndims, tile.t, tile.s1, tile.s2, tile.s3, h->R);
    cudaError_t e = cudaFuncSetAttribute((const void*)k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return cuda_fail(h, e);
    if (!j_rows(h, planes)) return STENCIL_OK;
    int occ = 1;
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, (const void*)k, thr, (size_t)smem);
    if (e != cudaSuccess) return cuda_fail(h, e);
    h->occ = std::max(occ, 1);
    std::vector<RowPlan> rows;
    plan_rows(h->ndims, dims, T, tile, rows, h->R);
    int64_t need = 0;
    for (auto& r : rows) {
        const int J = choose_J(h, r);
        if (J > 1) need = std::max<int64_t>(need, (int64_t)r.w * r.n2);
    }
    if (h->ndims == 2 && need > 0) {
        const int64_t fneed = need * tile.t * (int64_t)(tile.s1 + tile.t + 2) * 2;
        if (fneed > h->faceg_n) {
            drop_graphs(h);
            if (h->faceg) cudaFree(h->faceg);
            h->faceg = nullptr;
            h->faceg_n = 0;
            e = cudaMalloc(&h->faceg, fneed * sizeof(float));
            if (e != cudaSuccess) return cuda_fail(h, e);
            h->faceg_n = fneed;
        }
    }
    if (need > h->flags_n) {
        // the cached graphs captured the old flag pointer (memset node and kernel
        // parameters): they must not be replayed after the buffer moves
        drop_graphs(h);
        if (h->flags) cudaFree(h->flags);
        h->flags = nullptr;
        h->flags_n = 0;
        e = cudaMalloc(&h->flags, need * sizeof(unsigned));
        if (e != cudaSuccess) return cuda_fail(h, e);
        h->flags_n = need;
    }
    return STENCIL_OK;
}

// Enqueue the hexagon rows (a3) for a domain of extents dims whose level 0 is
// in plane0 (ring included) and whose ring is also present in plane1; the
// result (level T) lands in plane[T & 1].  Ring values are read from `ring`.
static int enqueue_rows(stencil_t h, const int64_t* dims, const float* ring, float* plane0, float* plane1,
                        int64_t T, stencil_tile tile, int G, int thr, cudaStream_t s, int64_t* launches,
                        std::vector<cudaEvent_t>* evs = nullptr, bool planes = false) {
    std::vector<RowPlan> rows;
    plan_rows(h->ndims, dims, T, tile, rows, h->R);
    hex_kernel_t k = get_hex_kernel(h->ndims, h->kind, h->mode, h->has_c, h->defw, tile.s2, h->ndims == 3 ? tile.s3 : 0);
    if (!k) return STENCIL_EINVAL;
    const int64_t smem = smem_bytes(h->ndims, tile.t, tile.s1, tile.s2, tile.s3, h->R);
    int64_t nl = 0;
    cudaError_t e;
    // 3D: thread blocks per slab J (pipelined along S2, flags in global memory);
    // all blocks of a launch must be co-resident when J > 1 (no deadlock).
    // Occupancy and the flag buffer come from prepare_rows (outside capture).
    if (j_rows(h, planes)) {
        int64_t need = 0;
        for (auto& r : rows) {
            r.J = choose_J(h, r);
            if (r.J > 1) need = std::max<int64_t>(need, (int64_t)r.w * r.n2);
        }
        if (need > h->flags_n) return STENCIL_EINVAL;   // prepare_rows was not called
        if (need > 0) {
            e = cudaMemsetAsync(h->flags, 0, need * sizeof(unsigned), s);
            if (e != cudaSuccess) return cuda_fail(h, e);
        }
    }
    HexParams p;
    memset(&p, 0, sizeof(p));
    p.in = ring;
    p.plane[0] = plane0;
    p.plane[1] = plane1;
    p.S1 = dims[0]; p.S2 = h->ndims >= 2 ? dims[1] : 1; p.S3 = h->ndims == 3 ? dims[2] : 1;
    p.T = T;
    p.tT = tile.t; p.tS1 = tile.s1; p.tS2 = tile.s2; p.tS3 = h->ndims == 3 ? tile.s3 : 0;
    p.G = G;
    p.P = 2 * tile.s1 + h->R * tile.t;
    p.R = h->R;
    for (int j = 0; j < kMaxPts; ++j) p.w[j] = h->w[j];
    p.c = h->c;
    p.kappa = h->kappa;
    p.flags = h->flags;
    p.faceg = h->faceg;
    p.compute_only = h->compute_only;
    for (auto& r : rows) {
        p.t0 = r.t0; p.xbase = r.xbase; p.tau_lo = r.tau_lo; p.tau_hi = r.tau_hi;
        p.n2 = r.n2; p.n3 = r.n3; p.J = r.J;
        p.epoch = (unsigned)(r.m + 2) << 16;
        void* args[] = {&p};
        if (evs) {
            cudaEvent_t a, b;
            cudaEventCreate(&a);
            cudaEventCreate(&b);
            evs->push_back(a);
            evs->push_back(b);
            cudaEventRecord(a, s);
        }
        e = cudaLaunchKernel((const void*)k, dim3((unsigned)(r.w * r.J)), dim3(thr), args, (size_t)smem, s);
        if (e != cudaSuccess) return cuda_fail(h, e);
        if (evs) cudaEventRecord(evs->back(), s);
        ++nl;
    }
    *launches = nl;
    return STENCIL_OK;
}

static int enqueue_wavefront(stencil_t h, const RunSpec& r, cudaStream_t s, int64_t* launches);

static int enqueue_spec(stencil_t h, const RunSpec& r, cudaStream_t s, int64_t* launches) {
    if (r.planes_mode == 2) return enqueue_wavefront(h, r, s, launches);
    const int64_t n = r.dims[0] * r.dims[1] * r.dims[2];
    int64_t nl = 0, nrows = 0;
    int rc;
    if (r.planes_mode == 0) {
        float* plane[2];
        plane[r.T & 1] = r.b;
        plane[1 - (r.T & 1)] = h->scratch;
        // a2: level 0 in plane 0, the fixed ring in plane 1 (readings R2/R3)
        launch_copy_full(r.a, plane[0], n, s); ++nl;
        launch_copy_ring(r.a, plane[1], r.dims[0], r.dims[1], r.dims[2], s, h->R); ++nl;
        rc = enqueue_rows(h, r.dims, r.a, plane[0], plane[1], r.T, r.tile, r.G, r.thr, s, &nrows, nullptr);
    } else {
        float* p0 = const_cast<float*>(r.a);
        launch_copy_ring(p0, r.b, r.dims[0], r.dims[1], r.dims[2], s, h->R); ++nl;
        rc = enqueue_rows(h, r.dims, p0, p0, r.b, r.T, r.tile, r.G, r.thr, s, &nrows, nullptr, true);
    }
    *launches = nl + nrows;
    return rc;
}

static bool same_spec(const RunSpec& x, const RunSpec& y) {
    return x.planes_mode == y.planes_mode && x.a == y.a && x.b == y.b && x.dims[0] == y.dims[0] &&
           x.dims[1] == y.dims[1] && x.dims[2] == y.dims[2] && x.T == y.T && x.tile.t == y.tile.t &&
           x.tile.s1 == y.tile.s1 && x.tile.s2 == y.tile.s2 && x.tile.s3 == y.tile.s3 && x.G == y.G &&
           x.thr == y.thr;
}

// Run a spec through the CUDA-graph cache (captured once per spec, replayed).
static int run_spec(stencil_t h, const RunSpec& r, cudaStream_t s) {
    int prc = r.planes_mode == 2 ? STENCIL_OK : prepare_rows(h, r.dims, r.T, r.tile, r.thr, r.planes_mode == 1);
    if (prc) return prc;
    const bool use_graph = getenv("HHC_NO_GRAPH") == nullptr && !h->compute_only;
    if (!use_graph) {
        int64_t nl = 0;
        int rc = enqueue_spec(h, r, s, &nl);
        h->last_launches = nl;
        if (rc) return rc;
        return cuda_fail(h, cudaGetLastError());
    }
    for (auto& g : h->graphs) {
        if (same_spec(g.spec, r)) {
            g.last_use = ++h->use_clock;
            h->last_launches = g.launches;
            return cuda_fail(h, cudaGraphLaunch(g.exec, s));
        }
    }
    // capture on the private stream, then launch on the caller's stream
    cudaGraph_t graph = nullptr;
    cudaError_t e = cudaStreamBeginCapture(h->cap_stream, cudaStreamCaptureModeThreadLocal);
    if (e != cudaSuccess) return cuda_fail(h, e);
    int64_t nl = 0;
    int rc = enqueue_spec(h, r, h->cap_stream, &nl);
    e = cudaStreamEndCapture(h->cap_stream, &graph);
    if (rc) { if (graph) cudaGraphDestroy(graph); return rc; }
    if (e != cudaSuccess) return cuda_fail(h, e);
    cudaGraphExec_t exec = nullptr;
    e = cudaGraphInstantiate(&exec, graph, 0);
    cudaGraphDestroy(graph);
    if (e != cudaSuccess) return cuda_fail(h, e);
    if (h->graphs.size() >= 32) {
        auto it = std::min_element(h->graphs.begin(), h->graphs.end(),
                                   [](const GraphEntry& a, const GraphEntry& b) { return a.last_use < b.last_use; });
        cudaGraphExecDestroy(it->exec);
        h->graphs.erase(it);
    }
    h->graphs.push_back(GraphEntry{r, exec, nl, ++h->use_clock});
    h->last_launches = nl;
    return cuda_fail(h, cudaGraphLaunch(exec, s));
}

extern "C" int stencil_run(stencil_t h, const float* d_in, float* d_out, int64_t T, stencil_tile tile,
                           int threads, void* cuda_stream) {
    if (!h) return STENCIL_EINVAL;
    if (h->sticky) return h->sticky;
    if (!d_in || !d_out || T < 0) return STENCIL_EINVAL;
    const int64_t n = h->nelem();
    if (d_out < d_in + n && d_in < d_out + n) return STENCIL_EINVAL;   // overlap
    cudaStream_t s = (cudaStream_t)cuda_stream;
    cudaSetDevice(h->device);
    if (T == 0) {
        h->last_launches = 1;
        launch_copy_full(d_in, d_out, n, s);
        return cuda_fail(h, cudaGetLastError());
    }
    RunSpec r;
    int rc = check_tile(h->ndims, tile, threads, h->smem_optin, &r.G, &r.thr, h->kind);
    if (rc) return rc;
    if (!h->scratch) {
        cudaError_t e = cudaMalloc(&h->scratch, n * sizeof(float));
        if (e != cudaSuccess) { h->scratch = nullptr; return STENCIL_ENOMEM; }
    }
    r.planes_mode = 0; r.a = d_in; r.b = d_out;
    for (int d = 0; d < 3; ++d) r.dims[d] = h->dims[d];
    r.T = T; r.tile = tile;
    if (h->ndims == 2) r.tile.s3 = 0;
    return run_spec(h, r, s);
}

extern "C" int stencil_run_planes(stencil_t h, int64_t rows, float* plane0, float* plane1, int64_t T,
                                  stencil_tile tile, int threads, void* cuda_stream) {
    if (!h) return STENCIL_EINVAL;
    if (h->sticky) return h->sticky;
    if (!plane0 || !plane1 || T < 1 || rows < 3) return STENCIL_EINVAL;
    RunSpec r;
    int rc = check_tile(h->ndims, tile, threads, h->smem_optin, &r.G, &r.thr, h->kind);
    if (rc) return rc;
    cudaSetDevice(h->device);
    r.planes_mode = 1; r.a = plane0; r.b = plane1;
    r.dims[0] = rows; r.dims[1] = h->dims[1]; r.dims[2] = h->dims[2];
    const int64_t n = r.dims[0] * r.dims[1] * r.dims[2];
    if (plane1 < plane0 + n && plane0 < plane1 + n) return STENCIL_EINVAL;
    r.T = T; r.tile = tile;
    if (h->ndims == 2) r.tile.s3 = 0;
    return run_spec(h, r, (cudaStream_t)cuda_stream);
}

extern "C" int stencil_run_host(stencil_t h, const float* h_in, float* h_out, int64_t T, stencil_tile tile,
                                int threads, void* cuda_stream) {
    if (!h || !h_in || !h_out) return STENCIL_EINVAL;
    if (h->sticky) return h->sticky;
    const int64_t n = h->nelem();
    cudaStream_t s = (cudaStream_t)cuda_stream;
    cudaSetDevice(h->device);
    if (!h->h_in_dev) {
        if (cudaMalloc(&h->h_in_dev, n * sizeof(float)) != cudaSuccess) { h->h_in_dev = nullptr; return STENCIL_ENOMEM; }
        if (cudaMalloc(&h->h_out_dev, n * sizeof(float)) != cudaSuccess) { h->h_out_dev = nullptr; return STENCIL_ENOMEM; }
    }
    cudaError_t e = cudaMemcpyAsync(h->h_in_dev, h_in, n * sizeof(float), cudaMemcpyHostToDevice, s);
    if (e != cudaSuccess) return cuda_fail(h, e);
    int rc = stencil_run(h, h->h_in_dev, h->h_out_dev, T, tile, threads, cuda_stream);
    if (rc) return rc;
    e = cudaMemcpyAsync(h_out, h->h_out_dev, n * sizeof(float), cudaMemcpyDeviceToHost, s);
    if (e != cudaSuccess) return cuda_fail(h, e);
    return cuda_fail(h, cudaStreamSynchronize(s));
}

// n independent problems from/to host buffers, pipelined over two device buffer
// pairs: the H2D copy of problem i+1 (own stream) and the D2H copy of problem i-1
// (own stream) overlap the HHC rows of problem i on cuda_stream.  Events order
// every buffer reuse: in[k] is refilled after the run that read it, out[k] is
// rewritten after its D2H.  Synchronises before returning.
extern "C" int stencil_run_host_batch(stencil_t h, int n, const float* const* h_in, float* const* h_out, int64_t T,
                                      stencil_tile tile, int threads, void* cuda_stream) {
    if (!h || n < 1 || !h_in || !h_out) return STENCIL_EINVAL;
    if (h->sticky) return h->sticky;
    for (int i = 0; i < n; ++i)
        if (!h_in[i] || !h_out[i]) return STENCIL_EINVAL;
    const int64_t n_el = h->nelem();
    const size_t bytes = (size_t)n_el * sizeof(float);
    cudaStream_t s = (cudaStream_t)cuda_stream;
    cudaSetDevice(h->device);
    if (!h->hb_dev[0][0]) {
        for (int k = 0; k < 2; ++k) {
            for (int j = 0; j < 2; ++j)
                if (cudaMalloc(&h->hb_dev[k][j], bytes) != cudaSuccess) { h->hb_dev[k][j] = nullptr; return STENCIL_ENOMEM; }
            if (cudaStreamCreateWithFlags(&h->hb_s[k], cudaStreamNonBlocking) != cudaSuccess) return STENCIL_ECUDA;
            for (int j = 0; j < 3; ++j)
                if (cudaEventCreateWithFlags(&h->hb_ev[k][j], cudaEventDisableTiming) != cudaSuccess) return STENCIL_ECUDA;
        }
    }
    cudaStream_t sin = h->hb_s[0], sout = h->hb_s[1];
    // per slot k: ev[k][0] = input copied, ev[k][1] = run done, ev[k][2] = output copied
    cudaError_t e = cudaSuccess;
    auto upload = [&](int i) {
        const int k = i & 1;
        if (i >= 2) cudaStreamWaitEvent(sin, h->hb_ev[k][1], 0);       // the run of i-2 read in[k]
        e = cudaMemcpyAsync(h->hb_dev[k][0], h_in[i], bytes, cudaMemcpyHostToDevice, sin);
        cudaEventRecord(h->hb_ev[k][0], sin);
    };
    cudaEventRecord(h->hb_ev[1][1], s);        // orders the first uploads after earlier work on s
    cudaStreamWaitEvent(sin, h->hb_ev[1][1], 0);
    upload(0);
    for (int i = 0; i < n && e == cudaSuccess; ++i) {
        const int k = i & 1;
        if (i + 1 < n) upload(i + 1);
        cudaStreamWaitEvent(s, h->hb_ev[k][0], 0);                     // input i on the device
        if (i >= 2) cudaStreamWaitEvent(s, h->hb_ev[k][2], 0);         // out[k] copied out (problem i-2)
        int rc = stencil_run(h, h->hb_dev[k][0], h->hb_dev[k][1], T, tile, threads, cuda_stream);
        if (rc) return rc;
        cudaEventRecord(h->hb_ev[k][1], s);
        cudaStreamWaitEvent(sout, h->hb_ev[k][1], 0);
        e = cudaMemcpyAsync(h_out[i], h->hb_dev[k][1], bytes, cudaMemcpyDeviceToHost, sout);
        cudaEventRecord(h->hb_ev[k][2], sout);
    }
    if (e != cudaSuccess) return cuda_fail(h, e);
    e = cudaStreamSynchronize(sout);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    return cuda_fail(h, e);
}

// ---- wavefront-parallel Jacobi-1D (reading W1)
static int check_wave_tile(stencil_tile t) {
    if (t.t < 1 || t.t > 1024 || t.s1 < 2 || t.s1 > 16384) return STENCIL_ETILE;
    return STENCIL_OK;
}

extern "C" int stencil_wavefront_info(const int64_t* dims, int64_t T, stencil_tile tile, int64_t* n_wavefronts,
                                      int64_t* n_tiles, int64_t* max_width) {
    if (!dims || dims[0] < 3 || T < 1) return STENCIL_EINVAL;
    if (int rc = check_wave_tile(tile)) return rc;
    std::vector<WaveLaunch> ws;
    wave1d_schedule(dims[0], T, tile.t, tile.s1, ws);
    int64_t tiles = 0, mx = 0;
    for (auto& w : ws) { tiles += w.n; mx = std::max(mx, w.n); }
    if (n_wavefronts) *n_wavefronts = (int64_t)ws.size();
    if (n_tiles) *n_tiles = tiles;
    if (max_width) *max_width = mx;
    return STENCIL_OK;
}

static int enqueue_wavefront(stencil_t h, const RunSpec& r, cudaStream_t s, int64_t* launches) {
    const int64_t n = r.dims[0];
    float* plane[2];
    plane[r.T & 1] = r.b;
    plane[1 - (r.T & 1)] = h->scratch;
    launch_copy_full(r.a, plane[0], n, s);                  // a2: level 0 in plane 0
    launch_copy_ring(r.a, plane[1], n, 1, 1, s);            // the two ring points in plane 1
    std::vector<WaveLaunch> ws;
    wave1d_schedule(n, r.T, r.tile.t, r.tile.s1, ws);
    WaveParams p;
    memset(&p, 0, sizeof(p));
    p.plane[0] = plane[0];
    p.plane[1] = plane[1];
    p.S = n; p.T = r.T; p.tT = r.tile.t; p.tS = r.tile.s1;
    for (int k = 0; k < 3; ++k) p.w[k] = h->w[k];
    p.c = h->c;
    for (auto& w : ws) {
        p.d = w.d; p.ia = w.ia;
        if (launch_wave1d(h->mode, h->has_c, h->defw, p, w.n, s)) return cuda_fail(h, cudaErrorLaunchFailure);
    }
    *launches = 2 + (int64_t)ws.size();
    return STENCIL_OK;
}

extern "C" int stencil_run_wavefront(stencil_t h, const float* d_in, float* d_out, int64_t T, stencil_tile tile,
                                     void* cuda_stream) {
    if (!h) return STENCIL_EINVAL;
    if (h->sticky) return h->sticky;
    if (h->kind != STENCIL_JACOBI1D_3PT || h->ndims != 1) return STENCIL_EINVAL;
    if (!d_in || !d_out || T < 0) return STENCIL_EINVAL;
    const int64_t n = h->nelem();
    if (d_out < d_in + n && d_in < d_out + n) return STENCIL_EINVAL;
    cudaStream_t s = (cudaStream_t)cuda_stream;
    cudaSetDevice(h->device);
    if (T == 0) {
        h->last_launches = 1;
        launch_copy_full(d_in, d_out, n, s);
        return cuda_fail(h, cudaGetLastError());
    }
    if (int rc = check_wave_tile(tile)) return rc;
    if (wave1d_smem_bytes(tile.t, tile.s1) > h->smem_optin) return STENCIL_ETILE;
    if (!h->scratch) {
        cudaError_t e = cudaMalloc(&h->scratch, n * sizeof(float));
        if (e != cudaSuccess) { h->scratch = nullptr; return STENCIL_ENOMEM; }
    }
    if (prepare_wave1d(h->mode, h->has_c, h->defw, tile.t, tile.s1)) return cuda_fail(h, cudaErrorInvalidValue);
    // through the CUDA-graph cache like stencil_run (one graph per pointers/T/tile)
    RunSpec r;
    memset(&r, 0, sizeof(r));
    r.planes_mode = 2; r.a = d_in; r.b = d_out;
    r.dims[0] = n; r.dims[1] = 1; r.dims[2] = 1;
    r.T = T; r.tile = tile; r.tile.s2 = r.tile.s3 = 0;
    r.G = 1; r.thr = 256;
    return run_spec(h, r, s);
}

extern "C" int64_t stencil_last_launches(stencil_t h) { return h ? h->last_launches : 0; }

extern "C" int stencil_profile(stencil_t h, const float* d_in, float* d_out, int64_t T, stencil_tile tile,
                               int threads, void* cuda_stream, double* kernel_seconds, int64_t* kernel_launches) {
    if (!h || !kernel_seconds || !kernel_launches) return STENCIL_EINVAL;
    if (h->sticky) return h->sticky;
    if (!d_in || !d_out || T < 1) return STENCIL_EINVAL;
    int G, thr;
    int rc = check_tile(h->ndims, tile, threads, h->smem_optin, &G, &thr, h->kind);
    if (rc) return rc;
    const int64_t n = h->nelem();
    if (!h->scratch) {
        if (cudaMalloc(&h->scratch, n * sizeof(float)) != cudaSuccess) { h->scratch = nullptr; return STENCIL_ENOMEM; }
    }
    cudaStream_t s = (cudaStream_t)cuda_stream;
    cudaSetDevice(h->device);
    float* plane[2];
    plane[T & 1] = d_out;
    plane[1 - (T & 1)] = h->scratch;
    launch_copy_full(d_in, plane[0], n, s);
    launch_copy_ring(d_in, plane[1], h->dims[0], h->dims[1], h->dims[2], s, h->R);
    rc = prepare_rows(h, h->dims, T, tile, thr);
    if (rc) return rc;
    std::vector<cudaEvent_t> evs;
    int64_t nl = 0;
    rc = enqueue_rows(h, h->dims, d_in, plane[0], plane[1], T, tile, G, thr, s, &nl, &evs);
    if (rc == STENCIL_OK) rc = cuda_fail(h, cudaStreamSynchronize(s));
    double tot = 0.0;
    for (size_t i = 0; i + 1 < evs.size(); i += 2) {
        float ms = 0.0f;
        if (rc == STENCIL_OK) cudaEventElapsedTime(&ms, evs[i], evs[i + 1]);
        tot += ms * 1e-3;
    }
    for (auto ev : evs) cudaEventDestroy(ev);
    *kernel_seconds = tot;
    *kernel_launches = (int64_t)(evs.size() / 2);
    return rc;
}

extern "C" int stencil_microbench(int which, stencil_kind kind, int ndims, const int64_t* dims, int64_t T,
                                  stencil_tile tile, int threads, double* value) {
    if (!value) return STENCIL_EINVAL;
    return run_microbench(which, kind, ndims, dims, T, tile, threads, value);
}

namespace hhc {
void set_compute_only(stencil_t h, int on) { if (h) h->compute_only = on; }

void set_last_launches(stencil_t h, int64_t n) { if (h) h->last_launches = n; }

int handle_radius(stencil_t h) { return h ? h->R : 1; }

void handle_info(stencil_t h, int* kind, int* ndims, int64_t* dims, int* device) {
    *kind = h->kind;
    *ndims = h->ndims;
    for (int d = 0; d < 3; ++d) dims[d] = h->dims[d];
    *device = h->device;
}

// A handle with h's stencil (kind, weights, c, mode) on other extents; maxJ > 0
// caps its 3D blocks per slab (the multi-GPU edge runs use 1: they never spin on
// progress flags, so they can share the GPU with a J-pipelined interior run).
int handle_clone(stencil_t h, const int64_t* dims, int maxJ, stencil_t* out) {
    float co[kMaxPts + 1];
    int n = 0;
    if (h->kind == STENCIL_GRADIENT2D) {
        co[n++] = h->kappa;
    } else {
        for (int j = 0; j < h->npts; ++j) co[n++] = h->w[j];
        co[n++] = h->c;
    }
    const int rc = stencil_create((stencil_kind)h->kind, h->ndims, dims, co, n, h->mode, out);
    if (rc == STENCIL_OK) (*out)->maxJ = maxJ;
    return rc;
}
}

// ---- f1: non-redundant, hexagon-aligned multi-GPU decomposition (2D).
// Hexagons are assigned to ranks by their centre column (owned rows [b0, b1) of
// the slab partition); every point is computed exactly once (no ghost rows, no
// redundant compute).  A rank stores the global rows [b0 - H, b1 + H) its
// hexagons touch (H = tS1/2 + tT/2 + 3: half a hexagon plus the footprint halo)
// in planes indexed by global x.  K1 writes every facet row that a neighbour
// also stores straight into the neighbour's plane (peer stores fused into the
// edge CTAs, HexParams::peer), so after row m of hexagons every value row m+1
// reads is in the reader's own planes.  Dependences: row m+1 on any rank reads
// only values of rows <= m (reading G2), so the rows are run in order, all
// ranks' hexagons of row m before row m+1.  stencil_run_hexdist_local runs
// `world` virtual ranks of one device this way (peer stores = device stores
// into the neighbour's buffers); across GPUs the same kernel stores through
// peer-mapped (IPC) pointers over NVLink.
namespace {
struct HexRank {
    int64_t b0, b1, x_lo, x_hi, held_lo, held_hi;
    float* P[2] = {nullptr, nullptr};
    float* Pg[2] = {nullptr, nullptr};
};
}  // namespace

extern "C" int stencil_hexdist_partition(int64_t S1, int rank, int world, stencil_tile tile, int64_t* part) {
    if (!part || S1 < 3 || world < 1 || rank < 0 || rank >= world || tile.t < 2 || tile.s1 < 1) return STENCIL_EINVAL;
    const int64_t own = cdiv(S1 - 2, world);
    const int64_t H = tile.s1 / 2 + tile.t / 2 + 3;
    if (world > 1 && own < 2 * H) return STENCIL_ETILE;
    const int64_t b0 = 1 + rank * own, b1 = std::min<int64_t>(1 + (rank + 1) * own, S1 - 1);
    if (b1 <= b0) return STENCIL_EINVAL;
    if (world > 1 && rank < world - 1 && b1 - b0 < 2 * H) return STENCIL_ETILE;
    const int64_t v[6] = {b0, b1, std::max<int64_t>(0, b0 - H), std::min<int64_t>(S1, b1 + H),
                          b0 - (rank == 0 ? 1 : 0), b1 + (rank == world - 1 ? 1 : 0)};
    memcpy(part, v, sizeof(v));
    return STENCIL_OK;
}

extern "C" int stencil_run_hexdist_local(stencil_t h, int world, const float* d_in, float* d_out, int64_t T,
                                         stencil_tile tile, int threads, void* cuda_stream) {
    if (!h || world < 1 || !d_in || !d_out || T < 1) return STENCIL_EINVAL;
    if (h->sticky) return h->sticky;
    if (h->ndims != 2) return STENCIL_EINVAL;                  // the facet peer stores are K1's
    int G, thr;
    if (int rc = check_tile(h->ndims, tile, threads, h->smem_optin, &G, &thr, h->kind)) return rc;
    cudaStream_t s = (cudaStream_t)cuda_stream;
    cudaSetDevice(h->device);
    const int64_t S1 = h->dims[0], S2 = h->dims[1], inner = S2;
    std::vector<HexRank> rk(world);
    auto release = [&]() {
        cudaStreamSynchronize(s);
        for (auto& r : rk)
            for (float* p : r.P)
                if (p) cudaFree(p);
    };
    for (int k = 0; k < world; ++k) {
        int64_t part[6];
        if (int rc = stencil_hexdist_partition(S1, k, world, tile, part)) { release(); return rc; }
        HexRank& r = rk[k];
        r.b0 = part[0]; r.b1 = part[1]; r.x_lo = part[2]; r.x_hi = part[3]; r.held_lo = part[4]; r.held_hi = part[5];
        const size_t bytes = (size_t)((r.x_hi - r.x_lo) * inner) * sizeof(float);
        for (int i = 0; i < 2; ++i) {
            if (cudaMalloc(&r.P[i], bytes) != cudaSuccess) { release(); return STENCIL_ENOMEM; }
            r.Pg[i] = r.P[i] - r.x_lo * inner;                 // global-x indexed
            // level 0 (and its ring) into both planes
            cudaMemcpyAsync(r.P[i], d_in + r.x_lo * inner, bytes, cudaMemcpyDeviceToDevice, s);
        }
    }
    if (int rc = prepare_rows(h, h->dims, T, tile, thr)) { release(); return rc; }
    hex_kernel_t kern = get_hex_kernel(h->ndims, h->kind, h->mode, h->has_c, h->defw, tile.s2, h->ndims == 3 ? tile.s3 : 0);
    const int64_t smem = smem_bytes(h->ndims, tile.t, tile.s1, tile.s2, tile.s3, h->R);
    std::vector<RowPlan> rows;
    plan_rows(h->ndims, h->dims, T, tile, rows, h->R);
    HexParams p;
    memset(&p, 0, sizeof(p));
    p.S1 = S1; p.S2 = S2; p.S3 = 1; p.T = T;
    p.tT = tile.t; p.tS1 = tile.s1; p.tS2 = tile.s2; p.tS3 = 0;
    p.G = G; p.P = 2 * tile.s1 + tile.t; p.R = 1; p.J = 1;
    for (int j = 0; j < kMaxPts; ++j) p.w[j] = h->w[j];
    p.c = h->c; p.kappa = h->kappa;
    int64_t nl = 0;
    for (auto& row : rows) {
        p.t0 = row.t0; p.tau_lo = row.tau_lo; p.tau_hi = row.tau_hi; p.n2 = row.n2; p.n3 = 1;
        for (int k = 0; k < world; ++k) {
            const HexRank& r = rk[k];
            // hexagons j of this row whose centre 2 x0 + tS1 lies in [2 b0, 2 b1)
            auto first_at = [&](int64_t b) {            // smallest j with 2(xbase + jP) + tS1 >= 2b
                const int64_t num = 2 * b - tile.s1 - 2 * row.xbase;
                return num <= 0 ? (int64_t)0 : cdiv(num, 2 * (int64_t)p.P);
            };
            const int64_t jlo = k == 0 ? 0 : std::min<int64_t>(first_at(r.b0), row.w);
            const int64_t jhi = k == world - 1 ? row.w : std::min<int64_t>(first_at(r.b1), row.w);
            if (jhi <= jlo) continue;
            p.xbase = row.xbase + jlo * p.P;
            p.in = r.Pg[0];
            p.plane[0] = r.Pg[0];
            p.plane[1] = r.Pg[1];
            p.npeer = world > 1;
            for (int sd = 0; sd < 2; ++sd) {
                const int nb = k + (sd == 0 ? -1 : 1);
                if (nb >= 0 && nb < world) {
                    p.peer[sd][0] = rk[nb].Pg[0]; p.peer[sd][1] = rk[nb].Pg[1];
                    p.peer_lo[sd] = rk[nb].x_lo; p.peer_hi[sd] = rk[nb].x_hi;
                } else {
                    p.peer[sd][0] = p.peer[sd][1] = nullptr;
                    p.peer_lo[sd] = p.peer_hi[sd] = 0;
                }
            }
            void* args[] = {&p};
            cudaError_t e = cudaLaunchKernel((const void*)kern, dim3((unsigned)(jhi - jlo)), dim3(thr), args,
                                             (size_t)smem, s);
            if (e != cudaSuccess) { release(); return cuda_fail(h, e); }
            ++nl;
        }
    }
    for (auto& r : rk) {
        const int64_t n = (r.held_hi - r.held_lo) * inner;
        cudaMemcpyAsync(d_out + r.held_lo * inner, r.Pg[T & 1] + r.held_lo * inner, (size_t)n * sizeof(float),
                        cudaMemcpyDeviceToDevice, s);
    }
    h->last_launches = nl;
    const int rc = cuda_fail(h, cudaGetLastError());
    release();
    return rc;
}

// ---- f1 across processes (one per GPU): the rank's planes and a flag pair are
// exported as CUDA IPC handles, the neighbours' ones are opened (peer-mapped over
// NVLink), K1 stores facets straight into them, and each row of hexagons waits
// on the device until both neighbours have finished the previous row (flag
// written by the neighbour's signal kernel with a system-scope release).
namespace {
__global__ void hexdist_wait_kernel(const volatile unsigned* flags, unsigned want0, unsigned want1) {
    if (threadIdx.x == 0) {
        while ((int)(flags[0] - want0) < 0) __nanosleep(100);
        while ((int)(flags[1] - want1) < 0) __nanosleep(100);
        __threadfence_system();
    }
}
__global__ void hexdist_signal_kernel(unsigned* lo, unsigned* hi, unsigned v) {
    if (threadIdx.x == 0) {
        __threadfence_system();
        if (lo) asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(lo), "r"(v) : "memory");
        if (hi) asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(hi), "r"(v) : "memory");
    }
}
}  // namespace

struct stencil_hexdist_s {
    int rank = 0, world = 1, device = 0;
    stencil_tile tile{};
    HexRank me;
    unsigned* flags = nullptr;            // [2]: written by the lower / upper neighbour
    float* peerP[2][2] = {{nullptr, nullptr}, {nullptr, nullptr}};   // opened IPC planes (raw)
    unsigned* peerF[2] = {nullptr, nullptr};                         // neighbour's flag slot for me
    int64_t peer_lo[2] = {0, 0}, peer_hi[2] = {0, 0};
    unsigned epoch = 0;
};

extern "C" int stencil_hexdist_create(stencil_t h, int rank, int world, stencil_tile tile, unsigned char handles[192],
                                      void** out) {
    if (!h || !handles || !out || h->ndims != 2) return STENCIL_EINVAL;
    *out = nullptr;
    int64_t part[6];
    if (int rc = stencil_hexdist_partition(h->dims[0], rank, world, tile, part)) return rc;
    cudaSetDevice(h->device);
    auto* d = new stencil_hexdist_s();
    d->rank = rank; d->world = world; d->device = h->device; d->tile = tile;
    HexRank& r = d->me;
    r.b0 = part[0]; r.b1 = part[1]; r.x_lo = part[2]; r.x_hi = part[3]; r.held_lo = part[4]; r.held_hi = part[5];
    const size_t bytes = (size_t)((r.x_hi - r.x_lo) * h->dims[1]) * sizeof(float);
    cudaIpcMemHandle_t hd[3];
    bool ok = cudaMalloc(&r.P[0], bytes) == cudaSuccess && cudaMalloc(&r.P[1], bytes) == cudaSuccess &&
              cudaMalloc(&d->flags, 2 * sizeof(unsigned)) == cudaSuccess &&
              cudaMemset(d->flags, 0, 2 * sizeof(unsigned)) == cudaSuccess &&
              cudaIpcGetMemHandle(&hd[0], r.P[0]) == cudaSuccess && cudaIpcGetMemHandle(&hd[1], r.P[1]) == cudaSuccess &&
              cudaIpcGetMemHandle(&hd[2], d->flags) == cudaSuccess;
    if (!ok) {
        if (r.P[0]) cudaFree(r.P[0]);
        if (r.P[1]) cudaFree(r.P[1]);
        if (d->flags) cudaFree(d->flags);
        delete d;
        cudaGetLastError();
        return STENCIL_ECUDA;
    }
    for (int i = 0; i < 2; ++i) r.Pg[i] = r.P[i] - r.x_lo * h->dims[1];
    memcpy(handles, hd, 3 * sizeof(cudaIpcMemHandle_t));
    *out = d;
    return STENCIL_OK;
}

// handles of the lower (rank-1) and upper (rank+1) neighbour; NULL where none
extern "C" int stencil_hexdist_connect(stencil_t h, void* hd, const unsigned char lo[192], const unsigned char hi[192]) {
    auto* d = static_cast<stencil_hexdist_s*>(hd);
    if (!h || !d) return STENCIL_EINVAL;
    cudaSetDevice(d->device);
    const unsigned char* src[2] = {lo, hi};
    for (int sd = 0; sd < 2; ++sd) {
        const int nb = d->rank + (sd == 0 ? -1 : 1);
        if (nb < 0 || nb >= d->world) continue;
        if (!src[sd]) return STENCIL_EINVAL;
        cudaIpcMemHandle_t hh[3];
        memcpy(hh, src[sd], sizeof(hh));
        void* ptr[3] = {nullptr, nullptr, nullptr};
        for (int i = 0; i < 3; ++i)
            if (cudaIpcOpenMemHandle(&ptr[i], hh[i], cudaIpcMemLazyEnablePeerAccess) != cudaSuccess) {
                cudaGetLastError();
                for (int j = 0; j < i; ++j) cudaIpcCloseMemHandle(ptr[j]);   // no half-open neighbour
                return STENCIL_ECUDA;
            }
        int64_t part[6];
        if (int rc = stencil_hexdist_partition(h->dims[0], nb, d->world, d->tile, part)) return rc;
        d->peer_lo[sd] = part[2];
        d->peer_hi[sd] = part[3];
        for (int i = 0; i < 2; ++i) d->peerP[sd][i] = static_cast<float*>(ptr[i]);
        // my slot in the neighbour's flag pair: I am its upper neighbour if sd == 0
        d->peerF[sd] = static_cast<unsigned*>(ptr[2]) + (sd == 0 ? 1 : 0);
    }
    return STENCIL_OK;
}

extern "C" void stencil_hexdist_destroy(void* hd) {
    auto* d = static_cast<stencil_hexdist_s*>(hd);
    if (!d) return;
    cudaSetDevice(d->device);
    cudaDeviceSynchronize();
    for (int sd = 0; sd < 2; ++sd) {
        if (d->peerP[sd][0]) cudaIpcCloseMemHandle(d->peerP[sd][0]);
        if (d->peerP[sd][1]) cudaIpcCloseMemHandle(d->peerP[sd][1]);
        if (d->peerF[sd]) cudaIpcCloseMemHandle(d->peerF[sd] - (sd == 0 ? 1 : 0));
    }
    if (d->me.P[0]) cudaFree(d->me.P[0]);
    if (d->me.P[1]) cudaFree(d->me.P[1]);
    if (d->flags) cudaFree(d->flags);
    delete d;
}

// A_T on this rank: d_in_slab / d_out_slab hold the rows [held_lo, held_hi) of
// stencil_hexdist_partition; d_in_slab must also cover the stored rows, so the
// caller passes the stored rows [x_lo, x_hi) of level 0 as d_in_stored.
extern "C" int stencil_run_hexdist(stencil_t h, void* hd, const float* d_in_stored, float* d_out_slab, int64_t T,
                                   int threads, void* cuda_stream) {
    auto* d = static_cast<stencil_hexdist_s*>(hd);
    if (!h || !d || !d_in_stored || !d_out_slab || T < 1) return STENCIL_EINVAL;
    if (h->sticky) return h->sticky;
    const stencil_tile tile = d->tile;
    int G, thr;
    if (int rc = check_tile(h->ndims, tile, threads, h->smem_optin, &G, &thr, h->kind)) return rc;
    cudaStream_t s = (cudaStream_t)cuda_stream;
    cudaSetDevice(h->device);
    const int64_t S1 = h->dims[0], S2 = h->dims[1];
    HexRank& r = d->me;
    const size_t bytes = (size_t)((r.x_hi - r.x_lo) * S2) * sizeof(float);
    for (int i = 0; i < 2; ++i) cudaMemcpyAsync(r.P[i], d_in_stored, bytes, cudaMemcpyDeviceToDevice, s);
    if (int rc = prepare_rows(h, h->dims, T, tile, thr)) return rc;
    hex_kernel_t kern = get_hex_kernel(h->ndims, h->kind, h->mode, h->has_c, h->defw, tile.s2, h->ndims == 3 ? tile.s3 : 0);
    const int64_t smem = smem_bytes(h->ndims, tile.t, tile.s1, tile.s2, tile.s3, h->R);
    std::vector<RowPlan> rows;
    plan_rows(h->ndims, h->dims, T, tile, rows, h->R);
    HexParams p;
    memset(&p, 0, sizeof(p));
    p.S1 = S1; p.S2 = S2; p.S3 = 1; p.T = T;
    p.tT = tile.t; p.tS1 = tile.s1; p.tS2 = tile.s2;
    p.G = G; p.P = 2 * tile.s1 + tile.t; p.R = 1; p.J = 1;
    for (int j = 0; j < kMaxPts; ++j) p.w[j] = h->w[j];
    p.c = h->c; p.kappa = h->kappa;
    p.in = r.Pg[0]; p.plane[0] = r.Pg[0]; p.plane[1] = r.Pg[1];
    p.npeer = d->world > 1;
    for (int sd = 0; sd < 2; ++sd) {
        for (int i = 0; i < 2; ++i) p.peer[sd][i] = d->peerP[sd][i] ? d->peerP[sd][i] - d->peer_lo[sd] * S2 : nullptr;
        p.peer_lo[sd] = d->peerP[sd][0] ? d->peer_lo[sd] : 0;
        p.peer_hi[sd] = d->peerP[sd][0] ? d->peer_hi[sd] : 0;
    }
    const bool lo = d->peerF[0] != nullptr, hi = d->peerF[1] != nullptr;
    int64_t nl = 2;
    // Epoch handshake (monotonic counters, Nw + 1 steps per run): step 1 = "my
    // planes hold this run's level 0" (signalled after the copies above, so a
    // neighbour's peer stores can never be overwritten by them, and only after
    // my previous run's output copy), step m + 1 = "my row m is done".  Row m
    // waits for both neighbours' step m.
    const unsigned base = d->epoch;
    if (lo || hi) {
        hexdist_signal_kernel<<<1, 32, 0, s>>>(d->peerF[0], d->peerF[1], base + 1);
        ++nl;
    }
    unsigned m = 0;
    for (auto& row : rows) {
        ++m;
        if (lo || hi) {
            hexdist_wait_kernel<<<1, 32, 0, s>>>(d->flags, lo ? base + m : 0u, hi ? base + m : 0u);
            ++nl;
        }
        p.t0 = row.t0; p.tau_lo = row.tau_lo; p.tau_hi = row.tau_hi; p.n2 = row.n2; p.n3 = 1;
        auto first_at = [&](int64_t b) {
            const int64_t num = 2 * b - tile.s1 - 2 * row.xbase;
            return num <= 0 ? (int64_t)0 : cdiv(num, 2 * (int64_t)p.P);
        };
        const int64_t jlo = d->rank == 0 ? 0 : std::min<int64_t>(first_at(r.b0), row.w);
        const int64_t jhi = d->rank == d->world - 1 ? row.w : std::min<int64_t>(first_at(r.b1), row.w);
        if (jhi > jlo) {
            p.xbase = row.xbase + jlo * p.P;
            void* args[] = {&p};
            cudaError_t e = cudaLaunchKernel((const void*)kern, dim3((unsigned)(jhi - jlo)), dim3(thr), args,
                                             (size_t)smem, s);
            if (e != cudaSuccess) return cuda_fail(h, e);
            ++nl;
        }
        if (lo || hi) {
            hexdist_signal_kernel<<<1, 32, 0, s>>>(d->peerF[0], d->peerF[1], base + m + 1);
            ++nl;
        }
    }
    d->epoch = base + m + 1;
    // the neighbours' last row may still store level-T facets of my rows: wait for it
    // before the output copy (and before the next run's level-0 copies)
    if (lo || hi) {
        hexdist_wait_kernel<<<1, 32, 0, s>>>(d->flags, lo ? base + m + 1 : 0u, hi ? base + m + 1 : 0u);
        ++nl;
    }
    const int64_t n = (r.held_hi - r.held_lo) * S2;
    cudaMemcpyAsync(d_out_slab, r.Pg[T & 1] + r.held_lo * S2, (size_t)n * sizeof(float), cudaMemcpyDeviceToDevice, s);
    h->last_launches = nl;
    return cuda_fail(h, cudaGetLastError());
}
