/*
 * hhc.h -- C ABI of the B200 HHC stencil library (libhhc.so).
 *
 * Implements the data-parallel hot path of Prajapati et al., "Simple,
 * Accurate, Analytical Time Modeling and Optimal Tile Size Selection for GPGPU
 * Stencils" (PPoPP'17).  Citations "P:Lnnn" are PAPER.md lines.
 *
 *   stencil_create / stencil_run  -- iterative stencil of Eq. 1
 *       (1D, 2D or 3D) time-stepped T times under hybrid hexagonal/classic (HHC) tiling
 *       (§3.1; Fig. 1-2): hexagons of base tS1 and height tT over
 *       (t, S1), classic time skewing over S2 (and S3), one kernel launch per
 *       row of hexagons, one thread block per hexagonal prism/slab
 *       sweeping its sub-tiles sequentially.
 *   model_predict      -- the analytical execution time Talg, Eqs. 2-30
 *                         (P:L556-1158).
 *   model_select_tile  -- Eq. 31 solved by exhaustive enumeration, plus the
 *                         "within 10% of Talg_min" candidates.
 *   stencil_run_planes -- one time tile of the slab-decomposed multi-GPU run
 *   stencil_run_dist   -- the multi-GPU slab path with its NCCL ghost exchange
 *                         (BASELINE.json north_star; not in the paper), see
 *                         DESIGN.md §8.
 *
 * Conventions (all functions):
 *   - Sizes are int64.  Arrays are fp32, contiguous, row-major, S1 OUTERMOST,
 *     the innermost dimension contiguous.
 *   - dims are the FULL extents including a one-cell fixed (Dirichlet) ring
 *     (reading R2, "boundary values are given"); the
 *     interior is [1, S_d-2] and only interior points are updated.
 *   - Functions return STENCIL_OK (0) or a negative stencil_status.
 *   - A handle is not thread-safe.  Asynchronous CUDA errors surface as
 *     STENCIL_ECUDA on the next call on that handle.
 */
#ifndef HHC_H
#define HHC_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    STENCIL_JACOBI2D_5PT = 1,      /* centre + 4 faces, weights 0.2 (reading R1)          */
    STENCIL_HEAT2D_9PT = 2,        /* 3x3 box, 1/4, 1/8, 1/16                               */
    STENCIL_GRADIENT2D = 3,        /* non-linear 5-point, kappa = 1/8                       */
    STENCIL_HEAT3D_7PT = 4,        /* centre + 6 faces, 1/4, 1/8                            */
    STENCIL_LAPLACIAN3D_27PT = 5,  /* 3x3x3 box, 1/2, 7/128, 3/256, 1/256                   */
    STENCIL_LAPLACIAN2D_5PT = 6,   /* centre + 4 faces, 1/2, 1/8                            */
    STENCIL_JACOBI1D_3PT = 7,      /* 1D: x-1, x, x+1, weights fp32(1/3) (the
                                      paper's Section 4.1 derivation)           */
    /* SURVEY §8(f) f4, higher-order stencils ("Generality": the hexagon
     * slopes and footprints change by constant factors): 1D radius-r binomial
     * smoothers, offsets -r..r, weights C(2r, r+d) / 4^r.  For these kinds the fixed
     * boundary ring is r cells wide (interior [r, S1-1-r]), hexagon rows widen by 2r
     * per level (pitch 2 tS1 + r tT), footprints/facets are 2r rows per side. */
    STENCIL_BINOM1D_R2 = 8,        /* 5-point,  1 4 6 4 1 / 16                              */
    STENCIL_BINOM1D_R3 = 9,        /* 7-point,  1 6 15 20 15 6 1 / 64                       */
    STENCIL_BINOM1D_R4 = 10        /* 9-point,  1 8 28 56 70 56 28 8 1 / 256                */
} stencil_kind;

typedef enum {
    STENCIL_OK = 0,
    STENCIL_EINVAL = -1,   /* bad kind/ndims/dims/pointer/coeffs/T/threads            */
    STENCIL_ETILE = -2,    /* tile violates Eq. 31's integrality or the smem limit   */
    STENCIL_ENOMEM = -3,   /* device or host allocation failed                        */
    STENCIL_ECUDA = -4,    /* a CUDA runtime error (sticky until stencil_destroy)     */
    STENCIL_ENCCL = -5,    /* NCCL missing or an NCCL call failed (multi-GPU path)    */
    STENCIL_ENODEV = -6    /* no usable sm_100 device                                 */
} stencil_status;

typedef enum { STENCIL_MODE_PLAIN = 0, STENCIL_MODE_FUSED = 1 } stencil_mode;

/* Tile sizes: the decision variables of Eq. 31.
 *   t  = tT  (even, >= 2), s1 = tS1 (>= 1), hexagon base along S1;
 *   2D: s2 = tS2, a multiple of 32 (inner, contiguous); s3 = 0.
 *   3D: s2 = tS2 >= 1 (middle), s3 = tS3, a multiple of 32 (inner).
 *   1D (Jacobi-1D): s2 = s3 = 0; 256 threads per hexagon. */
typedef struct { int32_t t, s1, s2, s3; } stencil_tile;

/* Table 1 hardware parameters (EH) + C_iter (CSH); Table 2-4. */
typedef struct {
    int32_t n_sm;              /* nSM                                                   */
    int32_t n_v;               /* nV, vector units (FP32 lanes) per SM                  */
    int32_t mtb_sm;            /* MTBSM, max thread blocks per SM                       */
    int32_t r_sm;              /* RSM, registers per SM                                 */
    int64_t m_sm_bytes;        /* MSM, shared memory per SM (bytes)                     */
    int64_t m_block_bytes;     /* shared memory per thread block (bytes)                */
    double  L_s_per_word;      /* L, time per 4-byte word of global memory access (s)   */
    double  tau_sync_s;        /* tau_sync, one block barrier (s)                       */
    double  T_sync_s;          /* T_sync, one host-GPU synchronisation / launch (s)     */
    double  C_iter_s;          /* C_iter, one loop-body iteration per vector unit (s)   */
    int32_t regs_per_thread;   /* 0 = unknown (paper); >0 bounds k in EXACT (Eq. 11)    */
    int32_t geometry;          /* 0 = PAPER-literal equations, 1 = EXACT (M1),
                                  2 = EXACT_G (+ x-group rows, M9), 3 = EXACT_GW (M9 +
                                  the x-groups' window prologue rows, M10)              */
    int32_t threads;           /* threads per block for EXACT k; 0 = library rule      */
    int32_t max_threads_sm;    /* resident threads per SM (EXACT k); 0 = 2048           */
    int32_t n_gpus;            /* >1: slab decomposition model (M7)           */
    double  link_bytes_per_s;  /* per-direction GPU-GPU bandwidth                       */
    double  link_latency_s;    /* per-message latency                                   */
    int32_t dist_overlap;      /* M7: 0 = exchange then the ghost-extended slab, 1 =
                                  edge sub-slabs overlapped with the interior           */
    double  window_rows;       /* geometry 3 (EXACT_GW, reading M10): row
                                  equivalents each x-group spends per level on its
                                  register window's prologue rows (fitted with C_iter
                                  and tau on the calibration instances); 0 elsewhere    */
} model_hw_params;

typedef struct stencil_s* stencil_t;     /* opaque; owned by the library */

/* Create a handle for one stencil problem on the CURRENT CUDA device.
 *   kind/ndims must agree (1D kind: ndims = 1; 2D kinds: ndims = 2; 3D kinds: ndims = 3);
 *   1D tiles are (t, s1, 0, 0): hexagons of base s1 (>= 1) and height t, 256 threads;
 *   dims[ndims] are full extents, each >= 3;
 *   coeffs == NULL -> the default weights of DESIGN.md R1.  Linear kinds take
 *   |N| weights in canonical (lexicographic offset) order, optionally followed
 *   by the constant c of Eq. 1 (ncoeffs = |N| or |N|+1).  Gradient takes {kappa}.
 *   mode: STENCIL_MODE_PLAIN (separately rounded mul/add) or FUSED (fma),
 *   see DESIGN.md R4.  The values are copied.  *out receives the handle. */
int stencil_create(stencil_kind kind, int ndims, const int64_t* dims,
                   const float* coeffs, int ncoeffs, int mode, stencil_t* out);

/* Release the handle, its scratch plane and its CUDA-graph cache.  NULL is a no-op. */
void stencil_destroy(stencil_t h);

/* A_T from A_0 = d_in (device pointers, Eq. 1 iterated T times).
 *   d_in is never written; d_out must not overlap d_in; both hold prod(dims)
 *   floats.  T >= 0 (T = 0 copies).  threads = 0 -> library rule, else a
 *   multiple of the tile's column threads (K1) and <= 1024.
 *   Stream-ordered and asynchronous on cuda_stream (a cudaStream_t, NULL =
 *   legacy default stream).  The handle owns one scratch plane (allocated on
 *   first use).  Rows of hexagons are captured once into a CUDA graph per
 *   (pointers, T, tile, threads, stream) and replayed. */
int stencil_run(stencil_t h, const float* d_in, float* d_out, int64_t T,
                stencil_tile tile, int threads, void* cuda_stream);

/* Like stencil_run but with HOST in/out buffers: copies in, runs, copies out,
 * synchronises (the end-to-end path bench.py's "e2e" measures). */
int stencil_run_host(stencil_t h, const float* h_in, float* h_out, int64_t T,
                     stencil_tile tile, int threads, void* cuda_stream);

/* n independent problems (same handle, T and tile) from/to HOST buffers h_in[i] ->
 * h_out[i] (n_elements floats each; pinned for overlap), pipelined: the
 * host-to-device copy of problem i+1 and the device-to-host copy of problem i-1
 * run on the library's own copy streams while problem i runs on cuda_stream
 * (two device buffer pairs, allocated at first use, owned by the handle).
 * Results as n calls of stencil_run_host.  Synchronises. */
int stencil_run_host_batch(stencil_t h, int n, const float* const* h_in, float* const* h_out, int64_t T,
                           stencil_tile tile, int threads, void* cuda_stream);

/* Predicted execution time Talg in seconds (Eqs. 2-30).
 * dims are full ABI extents (the model uses S = dims-2).  Returns NaN for
 * invalid arguments and +INFINITY for an infeasible tile (Eq. 31 constraints),
 * so min-searches skip it. */
double model_predict(stencil_kind kind, int ndims, const int64_t* dims, int64_t T,
                     stencil_tile tile, const model_hw_params* hw);

/* Eq. 31 by exhaustive enumeration: *best = argmin Talg (ties:
 * lexicographically smallest (t, s1, s2, s3)), *best_threads = the library's
 * threads rule, and the tiles with Talg <= (1+within)*Talg_min written to
 * cands[0..min(n, cap)) in enumeration order, *n_cands = n (may exceed cap).
 * Search space: DESIGN.md reading M6.  Returns STENCIL_ETILE if no tile is
 * feasible. */
int model_select_tile(stencil_kind kind, int ndims, const int64_t* dims, int64_t T,
                      const model_hw_params* hw, double within,
                      stencil_tile* best, int* best_threads,
                      stencil_tile* cands, int cap, int* n_cands);

/* Resources of the HHC kernel the library launches for (kind, ndims, tile,
 * threads, mode) with default weights: shared-memory bytes per block (Mtile,
 * Eq. 19 / reading M3), threads per block, and registers per thread from
 * cudaFuncGetAttributes -- the Rtile of Eq. 11 the paper could not know
 * (reading M4).  *regs_per_thread = 0 when kind = 0 or
 * no CUDA device is visible.  STENCIL_ETILE / STENCIL_EINVAL if the tile or
 * threads are invalid (then nothing is written).  Host only; no allocation. */
int stencil_tile_resources(stencil_kind kind, int ndims, stencil_tile tile, int threads, int mode,
                           int64_t* smem_bytes, int* block_threads, int* regs_per_thread);

/* Resident blocks per SM of that kernel (cudaOccupancyMaxActiveBlocksPerMultiprocessor
 * at its dynamic shared memory): the k of Eq. 11 as the hardware sees it,
 * against which the EXACT model's k is tested.  Needs a device (STENCIL_ENODEV). */
int stencil_tile_occupancy(stencil_kind kind, int ndims, stencil_tile tile, int threads, int mode,
                           int* blocks_per_sm);

/* Launch geometry of a run: number of hexagon rows (kernel launches, Nw) and
 * the number of thread blocks of phase-A and phase-B rows (w(i), Eq. 5). */
int stencil_plan_info(int ndims, const int64_t* dims, int64_t T, stencil_tile tile,
                      int64_t* n_rows, int64_t* w_a, int64_t* w_b, int64_t* n_sub);

/* Calibration micro-benchmarks (§5.2) on the current device.
 *   which: 0 = L (s per word, all SMs streaming), 1 = tau_sync (s per block
 *   barrier), 2 = T_sync (s per back-to-back launch), 3 = C_iter of `kind`
 *   at `tile` (compute-only kernel with global<->shared transfers removed).
 *   *value receives the measurement. */
int stencil_microbench(int which, stencil_kind kind, int ndims, const int64_t* dims,
                       int64_t T, stencil_tile tile, int threads, double* value);

/* One time tile of the multi-GPU slab path, also usable
 * alone: run T steps on a domain of `rows` x dims[1] (x dims[2]) whose level 0
 * (ring included) is in plane0 (device, read AND overwritten as scratch);
 * plane1 (device, same size, no overlap) receives the ring, then serves as the
 * second parity plane.  The result A_T is left in plane0 if T is even, plane1
 * if T is odd.  Inner extents come from the handle; rows may differ from
 * dims[0] (ghost-extended slabs).  Stream-ordered like stencil_run. */
int stencil_run_planes(stencil_t h, int64_t rows, float* plane0, float* plane1, int64_t T,
                       stencil_tile tile, int threads, void* cuda_stream);

/* ---- Multi-GPU slab path (BASELINE.json north_star -- the
 * paper is single-GPU, so no PAPER.md passage defines it; its time model is
 * DESIGN.md reading M7).  One process per GPU.  The interior S1 rows are cut
 * into `world` slabs of own = ceil((S1-2)/world) rows; every time tile of tT
 * steps each rank exchanges g = tT ghost rows with rank -/+ 1 by ncclSend /
 * ncclRecv inside ncclGroupStart/End (point to point, no collective), then runs
 * the HHC rows (stencil_run_planes) on its ghost-extended slab.  NCCL is
 * dlopen'ed (libnccl.so.2, the copy already loaded by the process if any). */

/* ncclGetUniqueId into id[128] (rank 0 calls it; the caller broadcasts it, e.g.
 * with torch.distributed).  STENCIL_ENCCL if NCCL cannot be loaded. */
int stencil_dist_get_unique_id(unsigned char id[128]);

/* ncclCommInitRank on `device` (made current).  *comm receives an opaque
 * communicator owned by the library (free with stencil_dist_destroy); it also
 * owns the ghost-extended planes, the edge buffers and a second stream.
 * world = 1 needs no id and no NCCL (with an id it still initialises a one-rank
 * NCCL communicator: the single-GPU test of the NCCL entry points). */
int stencil_dist_init(const unsigned char id[128], int rank, int world, int device, void** comm);

/* 0 (default): exchange, then the whole ghost-extended slab per tile (2g
 * redundant rows); 1: edge sub-slabs (3g rows per side) first on the second
 * stream, their owned rows sent at once, the ghost-free interior overlapped
 * with the exchange (6g redundant rows; used only if every slab holds >= 2g rows). */
int stencil_dist_set_overlap(void* comm, int overlap);

/* Synchronises the device, frees the communicator and its buffers.  NULL ok. */
void stencil_dist_destroy(void* comm);

/* Host-only slab geometry (no device needed): part[0..5] = owned rows [r0, r1),
 * ghost-extended rows [e0, e1), rows the caller's slab holds [held_lo, held_hi)
 * (owned + the physical ring row on rank 0 / world-1), global row indices.
 * STENCIL_ETILE if a slab is thinner than g (world > 1). */
int stencil_dist_partition(int64_t S1, int rank, int world, int64_t g, int64_t part[6]);

/* A_T on this rank's slab.  h was created with the GLOBAL dims.  d_in_slab and
 * d_out_slab (device, caller-owned, no overlap) hold rows [held_lo, held_hi) of
 * the global array (stencil_dist_partition with g = tile.t).  Every rank calls
 * it with the same T, tile and threads.  Stream-ordered on cuda_stream (the
 * NCCL operations too); returns before completion.  stencil_last_launches(h)
 * then counts this rank's kernel launches. */
int stencil_run_dist(stencil_t h, void* comm, const float* d_in_slab, float* d_out_slab, int64_t T,
                     stencil_tile tile, int threads, void* cuda_stream);

/* The same per-rank phases for `world` virtual ranks of ONE device in lock
 * step, the ghost exchange done by device copies from the neighbour's buffers:
 * full-grid d_in/d_out (every rank's held rows are written).  Synchronises.
 * The single-GPU test of the slab path. */
int stencil_run_dist_local(stencil_t h, int world, const float* d_in, float* d_out, int64_t T,
                           stencil_tile tile, int threads, int overlap, void* cuda_stream);

/* ---- non-redundant, hexagon-aligned multi-GPU decomposition (2D
 * kinds).  Hexagons go to ranks by their centre column (owned rows [b0, b1) =
 * the slab partition); every point is computed once.  A rank stores the global
 * rows [x_lo, x_hi) = [b0 - H, b1 + H) (H = tS1/2 + tT/2 + 3) its hexagons touch;
 * the K1 kernel writes each facet row (reading G3: a value some other hexagon
 * reads) that a neighbour also stores straight into the neighbour's plane (peer
 * stores from the edge CTAs, fused with the compute).  Rows of hexagons run in
 * order on all ranks (a row reads only earlier rows). */

/* part[0..5] = b0, b1, x_lo, x_hi, held_lo, held_hi of `rank` (host only);
 * STENCIL_ETILE if a slab holds fewer than 2H rows (a hexagon would reach two
 * ranks away). */
int stencil_hexdist_partition(int64_t S1, int rank, int world, stencil_tile tile, int64_t part[6]);

/* The f1 decomposition with `world` virtual ranks of ONE device (separate
 * planes per rank, peer stores = device stores into the neighbour's planes):
 * A_T from A_0 like stencil_run (full-grid device in/out, no overlap), 2D
 * handles only.  Synchronises.  stencil_last_launches(h) = the kernel launches
 * (rows x ranks). */
int stencil_run_hexdist_local(stencil_t h, int world, const float* d_in, float* d_out, int64_t T,
                              stencil_tile tile, int threads, void* cuda_stream);

/* f1 across processes (one per GPU, or several on one GPU for testing): this
 * rank's planes (stored rows) and a flag pair are allocated on the current
 * device and exported as three CUDA IPC handles (handles[192]); *out = an
 * opaque object (free with stencil_hexdist_destroy). */
int stencil_hexdist_create(stencil_t h, int rank, int world, stencil_tile tile, unsigned char handles[192],
                           void** out);
/* Open the lower (rank-1) and upper (rank+1) neighbours' handles (NULL where
 * there is none): their planes become peer-mapped targets of K1's facet stores,
 * their flag pair the target of this rank's row signals. */
int stencil_hexdist_connect(stencil_t h, void* hd, const unsigned char lo[192], const unsigned char hi[192]);
/* A_T on this rank.  d_in_stored holds level 0 of the stored rows [x_lo, x_hi),
 * d_out_slab receives the held rows [held_lo, held_hi) (stencil_hexdist_partition).
 * Every row of hexagons waits on the device (a spin kernel, acquire.sys) until
 * both neighbours finished the previous row and signals its own completion
 * (release.sys store into their flags); all ranks call it with the same T.
 * Stream-ordered; returns before completion. */
int stencil_run_hexdist(stencil_t h, void* hd, const float* d_in_stored, float* d_out_slab, int64_t T,
                        int threads, void* cuda_stream);
void stencil_hexdist_destroy(void* hd);

/* Measurement helper (bench.py roofline): run like stencil_run but without the
 * CUDA graph, with a CUDA event pair around every hexagon-row launch on
 * cuda_stream; synchronises and returns the summed device time of the HHC
 * kernel launches (*kernel_seconds) and their number (*kernel_launches). */
int stencil_profile(stencil_t h, const float* d_in, float* d_out, int64_t T, stencil_tile tile,
                    int threads, void* cuda_stream, double* kernel_seconds, int64_t* kernel_launches);

/* ---- Wavefront-parallel Jacobi-1D (reading W1).
 * The paper's generality claim, P:L1160-1170 ("Consider, wavefront parallel
 * Jacobi1D stencil. The total execution time is the sum of the times for each
 * wavefront ... equation 6 holds for wavefront parallel codes"): a second
 * schedule of the same Eq. 1 update.  Parallelogram tiles of tile.t levels x
 * tile.s1 columns in skewed coordinates x' = x + t; tile (i, j) covers the
 * levels (i*t, min((i+1)*t, T)] and x' in [j*s1, (j+1)*s1); one kernel launch
 * per anti-diagonal i + j (the wavefront), one thread block per tile.
 * tile.t in [1, 1024] (any parity), tile.s1 in [2, 16384]; s2, s3 ignored. */

/* A_T from A_0 like stencil_run (same pointer rules, stream-ordered,
 * asynchronous, scratch plane owned by the handle), on a handle created for
 * STENCIL_JACOBI1D_3PT (else STENCIL_EINVAL).  One launch per wavefront plus
 * two set-up copies, captured once into a CUDA graph per (pointers, T, tile)
 * and replayed, like stencil_run. */
int stencil_run_wavefront(stencil_t h, const float* d_in, float* d_out, int64_t T,
                          stencil_tile tile, void* cuda_stream);

/* Schedule of a wavefront run on dims[0] points: number of wavefronts
 * (launches), tiles in total and in the widest wavefront (host only). */
int stencil_wavefront_info(const int64_t* dims, int64_t T, stencil_tile tile,
                           int64_t* n_wavefronts, int64_t* n_tiles, int64_t* max_width);

/* Talg of the wavefront schedule in seconds: Eq. 6 summed per wavefront, each
 * with its own tile count, Ttile by Eqs. 8-12 on the parallelogram's
 * footprint (reading W1).  hw->geometry selects L per word (PAPER)
 * or per SM (EXACT, reading M5).  NaN for invalid arguments, +INFINITY for a
 * tile that does not fit m_block_bytes. */
double model_predict_wavefront(stencil_kind kind, int ndims, const int64_t* dims, int64_t T,
                               stencil_tile tile, const model_hw_params* hw);

/* Eq. 31 for the wavefront schedule (reading W3): *best = argmin of
 * model_predict_wavefront over t in [1, min(T, 128)] and s1 in {4, 6, 8, 12,
 * 16, 24, ...} (powers of two and 1.5x) up to min(16384, S + T rounded up to 4);
 * ties -> smallest (t, s1).  Tiles with Talg <= (1+within) Talg_min go to
 * cands[0..min(n, cap)) in enumeration order (t outer), *n_cands = n.
 * STENCIL_EINVAL for bad arguments, STENCIL_ETILE if nothing fits. */
int model_select_wavefront_tile(stencil_kind kind, int ndims, const int64_t* dims, int64_t T,
                                const model_hw_params* hw, double within, stencil_tile* best,
                                stencil_tile* cands, int cap, int* n_cands);

/* Human-readable status. */
const char* stencil_strerror(int status);

/* Number of kernel launches the last stencil_run / stencil_run_planes on h
 * issued (for the bench's gpu_launches claim). */
int64_t stencil_last_launches(stencil_t h);

#ifdef __cplusplus
}
#endif
#endif /* HHC_H */
