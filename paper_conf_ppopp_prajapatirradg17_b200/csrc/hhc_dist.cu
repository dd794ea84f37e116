// hhc_dist.cu -- the multi-GPU slab path of include/hhc.h (SURVEY §8(b) and
// §8(e); BASELINE.json north_star -- the paper itself is single-GPU).
//
// The interior S1 rows are cut into `world` contiguous slabs (own = ceil((S1-2)/
// world) rows, the edge ranks also hold the physical ring row).  Every time
// tile of Tt <= g = tT steps each rank exchanges g ghost rows with rank -/+ 1
// (ncclSend/ncclRecv inside ncclGroupStart/End: point to point, no collective)
// and runs the HHC rows on its ghost-extended slab, whose outermost rows act as
// a fixed ring for the tile; after Tt steps the owned rows are exact because
// the dependence cone of a radius-1 stencil grows one row per step.
//
//   plain   : exchange, then the whole extended slab (2g redundant rows per tile)
//   overlap : the two edge sub-slabs (3g rows around each neighbour side, fresh
//             ghosts included) run first on a second stream with a J = 1 handle
//             (no progress-flag waits, so they can share the GPU with the
//             J-pipelined interior), their exact owned rows go to the neighbours
//             at once, while the ghost-free interior sub-slab runs on the caller's
//             stream; the tile result is the interior plane with the edge rows and
//             the received ghosts copied in (6g redundant rows per tile).
//
// NCCL is loaded with dlopen (the copy torch already loaded, else the system
// one), so libhhc.so has no link-time NCCL dependency.  A second transport,
// stencil_run_dist_local, runs `world` virtual ranks of one device in lock step
// through the same per-rank phases with device copies in place of NCCL: it is
// how the slab path is tested on a single GPU.
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <nccl.h>

#include <algorithm>
#include <cstring>
#include <vector>

#include "hhc_internal.h"

namespace {

struct NcclApi {
    bool ok = false;
    ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
    ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
    ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
    ncclResult_t (*Send)(const void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*Recv)(void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*GroupStart)() = nullptr;
    ncclResult_t (*GroupEnd)() = nullptr;
};

NcclApi load_nccl() {
    NcclApi a;
    void* lib = dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);        // torch's copy, if loaded
    if (!lib) lib = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!lib) lib = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
    if (!lib) return a;
    a.GetUniqueId = (decltype(a.GetUniqueId))dlsym(lib, "ncclGetUniqueId");
    a.CommInitRank = (decltype(a.CommInitRank))dlsym(lib, "ncclCommInitRank");
    a.CommDestroy = (decltype(a.CommDestroy))dlsym(lib, "ncclCommDestroy");
    a.Send = (decltype(a.Send))dlsym(lib, "ncclSend");
    a.Recv = (decltype(a.Recv))dlsym(lib, "ncclRecv");
    a.GroupStart = (decltype(a.GroupStart))dlsym(lib, "ncclGroupStart");
    a.GroupEnd = (decltype(a.GroupEnd))dlsym(lib, "ncclGroupEnd");
    a.ok = a.GetUniqueId && a.CommInitRank && a.CommDestroy && a.Send && a.Recv && a.GroupStart && a.GroupEnd;
    return a;
}

NcclApi& nccl() {
    static NcclApi a = load_nccl();
    return a;
}

inline int64_t cdiv(int64_t a, int64_t b) { return (a + b - 1) / b; }

// Slab of one rank (global row indices): owned interior rows [r0, r1), the rows
// the caller's in/out slab holds [held_lo, held_hi) (owned + the physical ring
// row on the edge ranks), and the ghost-extended rows [e0, e1).
struct Part {
    int64_t r0, r1, e0, e1, held_lo, held_hi;
};

int partition(int64_t S1, int rank, int world, int64_t g, Part* p) {
    if (S1 < 3 || world < 1 || rank < 0 || rank >= world || g < 1) return STENCIL_EINVAL;
    const int64_t own = cdiv(S1 - 2, world);
    p->r0 = 1 + rank * own;
    p->r1 = std::min<int64_t>(1 + (rank + 1) * own, S1 - 1);
    if (p->r1 <= p->r0) return STENCIL_EINVAL;                      // rank owns no rows
    if (world > 1 && (own < g || (rank < world - 1 && p->r1 - p->r0 < g))) return STENCIL_ETILE;
    p->e0 = std::max<int64_t>(0, p->r0 - g);
    p->e1 = std::min<int64_t>(S1, p->r1 + g);
    p->held_lo = p->r0 - (rank == 0 ? 1 : 0);
    p->held_hi = p->r1 + (rank == world - 1 ? 1 : 0);
    return STENCIL_OK;
}

// Per-rank buffers and phases (shared by the NCCL and the local transport).
struct Rank {
    int rank = 0, world = 1;
    Part part{};
    int64_t g = 0, inner = 0, rows = 0, lo = 0, hi = 0;   // lo/hi: local owned rows
    bool up = false, dn = false, overlap = false;
    float* P[2] = {nullptr, nullptr};                     // ghost-extended planes
    float* Eu[2] = {nullptr, nullptr};                    // edge sub-slabs (3g rows)
    float* Ed[2] = {nullptr, nullptr};
    float* Ru = nullptr;                                  // received ghosts (overlap)
    float* Rd = nullptr;
    stencil_t he = nullptr;                               // edge handle, J = 1
    int64_t launches = 0;

    float* row(float* p, int64_t r) const { return p + r * inner; }
    size_t bytes(int64_t nrows) const { return (size_t)(nrows * inner) * sizeof(float); }

    void release() {
        for (float* p : {P[0], P[1], Eu[0], Eu[1], Ed[0], Ed[1], Ru, Rd})
            if (p) cudaFree(p);
        P[0] = P[1] = Eu[0] = Eu[1] = Ed[0] = Ed[1] = Ru = Rd = nullptr;
        if (he) stencil_destroy(he);
        he = nullptr;
    }

    int setup(stencil_t h, int rk, int wd, int64_t gg, bool ovl) {
        int kind, nd, dev;
        int64_t dims[3];
        hhc::handle_info(h, &kind, &nd, dims, &dev);
        if (hhc::handle_radius(h) != 1) return STENCIL_EINVAL;   // slabs: radius-1 kinds (ring of one row)
        rank = rk; world = wd; g = gg;
        if (int rc = partition(dims[0], rank, world, g, &part)) return rc;
        inner = dims[1] * dims[2];
        rows = part.e1 - part.e0;
        lo = part.r0 - part.e0;
        hi = part.r1 - part.e0;
        up = rank > 0;
        dn = rank < world - 1;
        // one decision for all ranks (the NCCL pattern must match): every slab,
        // the last and thinnest included, holds at least 2g owned rows
        const int64_t own = cdiv(dims[0] - 2, world), last_own = dims[0] - 2 - (world - 1) * own;
        overlap = ovl && world > 1 && own >= 2 * g && last_own >= 2 * g;
        for (int i = 0; i < 2; ++i)
            if (cudaMalloc(&P[i], bytes(rows)) != cudaSuccess) return STENCIL_ENOMEM;
        if (overlap) {
            for (int i = 0; i < 2; ++i) {
                if (up && cudaMalloc(&Eu[i], bytes(3 * g)) != cudaSuccess) return STENCIL_ENOMEM;
                if (dn && cudaMalloc(&Ed[i], bytes(3 * g)) != cudaSuccess) return STENCIL_ENOMEM;
            }
            if (up && cudaMalloc(&Ru, bytes(g)) != cudaSuccess) return STENCIL_ENOMEM;
            if (dn && cudaMalloc(&Rd, bytes(g)) != cudaSuccess) return STENCIL_ENOMEM;
            const int64_t edims[3] = {3 * g, dims[1], dims[2]};
            if (int rc = hhc::handle_clone(h, edims, 1, &he)) return rc;
        }
        return STENCIL_OK;
    }

    int planes(stencil_t hh, int64_t nrows, float* a, float* b, int64_t Tt, stencil_tile tile, int thr,
               cudaStream_t s) {
        const int rc = stencil_run_planes(hh, nrows, a, b, Tt, tile, thr, s);
        launches += stencil_last_launches(hh);
        return rc;
    }
};

// The exchange of one rank: pairs (send, recv) per neighbour side.
struct Xfer {
    const float* up_send = nullptr;
    float* up_recv = nullptr;
    const float* dn_send = nullptr;
    float* dn_recv = nullptr;
};

Xfer plain_xfer(Rank& r, float* cur) {
    Xfer x;
    if (r.up) { x.up_send = r.row(cur, r.lo); x.up_recv = r.row(cur, r.lo - r.g); }
    if (r.dn) { x.dn_send = r.row(cur, r.hi - r.g); x.dn_recv = r.row(cur, r.hi); }
    return x;
}

// edge results of this tile: rows [g, 2g) of the edge sub-slab's result plane
Xfer edge_xfer(Rank& r, int64_t Tt) {
    Xfer x;
    const int k = (int)(Tt & 1);
    if (r.up) { x.up_send = r.row(r.Eu[k], r.g); x.up_recv = r.Ru; }
    if (r.dn) { x.dn_send = r.row(r.Ed[k], r.g); x.dn_recv = r.Rd; }
    return x;
}

}  // namespace

struct stencil_comm_s {
    int rank = 0, world = 1, device = 0;
    ncclComm_t nc = nullptr;
    int overlap = 0;
    Rank st;
    stencil_t bound = nullptr;     // handle the buffers were set up for
    int64_t bound_g = 0;
    int bound_overlap = -1;
    cudaStream_t s2 = nullptr;
    cudaEvent_t ev_a = nullptr, ev_b = nullptr;
};

namespace {

int nccl_exchange(stencil_comm_s* c, const Xfer& x, size_t n, cudaStream_t s) {
    NcclApi& a = nccl();
    if (a.GroupStart() != ncclSuccess) return STENCIL_ENCCL;
    bool bad = false;
    if (x.up_send) {
        bad |= a.Send(x.up_send, n, ncclFloat32, c->rank - 1, c->nc, s) != ncclSuccess;
        bad |= a.Recv(x.up_recv, n, ncclFloat32, c->rank - 1, c->nc, s) != ncclSuccess;
    }
    if (x.dn_send) {
        bad |= a.Send(x.dn_send, n, ncclFloat32, c->rank + 1, c->nc, s) != ncclSuccess;
        bad |= a.Recv(x.dn_recv, n, ncclFloat32, c->rank + 1, c->nc, s) != ncclSuccess;
    }
    if (a.GroupEnd() != ncclSuccess || bad) return STENCIL_ENCCL;
    return STENCIL_OK;
}

int cuda_rc(cudaError_t e) {
    return e == cudaSuccess ? STENCIL_OK : (e == cudaErrorMemoryAllocation ? STENCIL_ENOMEM : STENCIL_ECUDA);
}

// Overlap phase 1 of a tile: edge inputs copied out of cur (on s1, before the
// interior overwrites the other plane), edge runs on s2.
int edge_phase(Rank& r, float* cur, int64_t Tt, stencil_tile tile, int thr, cudaStream_t s1, cudaStream_t s2,
               cudaEvent_t ev) {
    cudaError_t e = cudaSuccess;
    if (r.up) e = cudaMemcpyAsync(r.Eu[0], r.row(cur, r.lo - r.g), r.bytes(3 * r.g), cudaMemcpyDeviceToDevice, s1);
    if (e == cudaSuccess && r.dn)
        e = cudaMemcpyAsync(r.Ed[0], r.row(cur, r.hi - 2 * r.g), r.bytes(3 * r.g), cudaMemcpyDeviceToDevice, s1);
    if (e != cudaSuccess) return cuda_rc(e);
    if (s2 != s1) {
        cudaEventRecord(ev, s1);
        cudaStreamWaitEvent(s2, ev, 0);
    }
    if (r.up)
        if (int rc = r.planes(r.he, 3 * r.g, r.Eu[0], r.Eu[1], Tt, tile, thr, s2)) return rc;
    if (r.dn)
        if (int rc = r.planes(r.he, 3 * r.g, r.Ed[0], r.Ed[1], Tt, tile, thr, s2)) return rc;
    return STENCIL_OK;
}

// Overlap phase 2: the ghost-free interior sub-slab (owned rows; the physical
// ring row on an edge rank) on s1; its result plane is cur (Tt even) or oth.
int interior_phase(Rank& r, stencil_t h, float* cur, float* oth, int64_t Tt, stencil_tile tile, int thr,
                   cudaStream_t s1) {
    const int64_t A = r.up ? r.lo : 0, B = r.dn ? r.hi : r.rows;
    return r.planes(h, B - A, r.row(cur, A), r.row(oth, A), Tt, tile, thr, s1);
}

// Overlap phase 3: assemble the tile result (on s1, after s2's edge runs and exchange).
int assemble_phase(Rank& r, float* res, int64_t Tt, bool last, cudaStream_t s1) {
    const int k = (int)(Tt & 1);
    cudaError_t e = cudaSuccess;
    if (r.up) {
        e = cudaMemcpyAsync(r.row(res, r.lo), r.row(r.Eu[k], r.g), r.bytes(r.g), cudaMemcpyDeviceToDevice, s1);
        if (e == cudaSuccess && !last)
            e = cudaMemcpyAsync(r.row(res, r.lo - r.g), r.Ru, r.bytes(r.g), cudaMemcpyDeviceToDevice, s1);
    }
    if (e == cudaSuccess && r.dn) {
        e = cudaMemcpyAsync(r.row(res, r.hi - r.g), r.row(r.Ed[k], r.g), r.bytes(r.g), cudaMemcpyDeviceToDevice, s1);
        if (e == cudaSuccess && !last)
            e = cudaMemcpyAsync(r.row(res, r.hi), r.Rd, r.bytes(r.g), cudaMemcpyDeviceToDevice, s1);
    }
    return cuda_rc(e);
}

}  // namespace

namespace {

int bind(stencil_comm_s* c, stencil_t h, stencil_tile tile) {
    const int ovl = c->overlap ? 1 : 0;
    if (c->bound == h && c->bound_g == tile.t && c->bound_overlap == ovl) return STENCIL_OK;
    c->st.release();
    c->bound = nullptr;
    const int rc = c->st.setup(h, c->rank, c->world, tile.t, ovl != 0);
    if (rc) { c->st.release(); return rc; }
    c->bound = h;
    c->bound_g = tile.t;
    c->bound_overlap = ovl;
    return STENCIL_OK;
}

}  // namespace

extern "C" int stencil_dist_partition(int64_t S1, int rank, int world, int64_t g, int64_t* part) {
    if (!part) return STENCIL_EINVAL;
    Part p;
    if (int rc = partition(S1, rank, world, g, &p)) return rc;
    const int64_t v[6] = {p.r0, p.r1, p.e0, p.e1, p.held_lo, p.held_hi};
    memcpy(part, v, sizeof(v));
    return STENCIL_OK;
}

extern "C" int stencil_dist_get_unique_id(unsigned char id[128]) {
    static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId is 128 bytes");
    if (!id) return STENCIL_EINVAL;
    if (!nccl().ok) return STENCIL_ENCCL;
    ncclUniqueId u;
    if (nccl().GetUniqueId(&u) != ncclSuccess) return STENCIL_ENCCL;
    memcpy(id, &u, sizeof(u));
    return STENCIL_OK;
}

extern "C" int stencil_dist_init(const unsigned char id[128], int rank, int world, int device, void** comm) {
    if (!comm || world < 1 || rank < 0 || rank >= world) return STENCIL_EINVAL;
    *comm = nullptr;
    if (cudaSetDevice(device) != cudaSuccess) return STENCIL_ENODEV;
    stencil_comm_s* c = new stencil_comm_s();
    c->rank = rank; c->world = world; c->device = device;
    // NCCL for world > 1; at world 1 only when an id is given (the single-GPU test of
    // the dlopen'ed NCCL entry points: unique id, communicator init and destroy)
    if (world > 1 || id) {
        if (!id || !nccl().ok) { delete c; return STENCIL_ENCCL; }
        ncclUniqueId u;
        memcpy(&u, id, sizeof(u));
        if (nccl().CommInitRank(&c->nc, world, u, rank) != ncclSuccess) { delete c; return STENCIL_ENCCL; }
    }
    if (cudaStreamCreateWithFlags(&c->s2, cudaStreamNonBlocking) != cudaSuccess ||
        cudaEventCreateWithFlags(&c->ev_a, cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreateWithFlags(&c->ev_b, cudaEventDisableTiming) != cudaSuccess) {
        if (c->nc) nccl().CommDestroy(c->nc);
        delete c;
        return STENCIL_ECUDA;
    }
    *comm = c;
    return STENCIL_OK;
}

extern "C" int stencil_dist_set_overlap(void* comm, int overlap) {
    if (!comm || overlap < 0 || overlap > 1) return STENCIL_EINVAL;
    static_cast<stencil_comm_s*>(comm)->overlap = overlap;
    return STENCIL_OK;
}

extern "C" void stencil_dist_destroy(void* comm) {
    stencil_comm_s* c = static_cast<stencil_comm_s*>(comm);
    if (!c) return;
    cudaSetDevice(c->device);
    cudaDeviceSynchronize();
    c->st.release();
    if (c->nc) nccl().CommDestroy(c->nc);
    if (c->s2) cudaStreamDestroy(c->s2);
    if (c->ev_a) cudaEventDestroy(c->ev_a);
    if (c->ev_b) cudaEventDestroy(c->ev_b);
    delete c;
}

extern "C" int stencil_run_dist(stencil_t h, void* comm, const float* d_in_slab, float* d_out_slab, int64_t T,
                                stencil_tile tile, int threads, void* cuda_stream) {
    stencil_comm_s* c = static_cast<stencil_comm_s*>(comm);
    if (!h || !c || !d_in_slab || !d_out_slab || T < 1) return STENCIL_EINVAL;
    if (c->world > 1 && !c->nc) return STENCIL_ENCCL;
    if (int rc = bind(c, h, tile)) return rc;
    Rank& r = c->st;
    r.launches = 0;
    cudaStream_t s1 = (cudaStream_t)cuda_stream;
    const Part& p = r.part;
    const int64_t off = p.held_lo - p.e0;
    cudaError_t e = cudaMemcpyAsync(r.row(r.P[0], off), d_in_slab, r.bytes(p.held_hi - p.held_lo),
                                    cudaMemcpyDeviceToDevice, s1);
    if (e != cudaSuccess) return cuda_rc(e);
    const size_t n = (size_t)(r.g * r.inner);
    int ci = 0;
    int64_t done = 0;
    if (r.overlap) {
        if (int rc = nccl_exchange(c, plain_xfer(r, r.P[0]), n, s1)) return rc;     // ghosts of tile 0
    }
    while (done < T) {
        const int64_t Tt = std::min<int64_t>(tile.t, T - done);
        const bool last = done + Tt >= T;
        float* cur = r.P[ci];
        float* oth = r.P[1 - ci];
        int rc;
        if (!r.overlap) {
            if (c->world > 1 && (rc = nccl_exchange(c, plain_xfer(r, cur), n, s1))) return rc;
            if ((rc = r.planes(h, r.rows, cur, oth, Tt, tile, threads, s1))) return rc;
        } else {
            if ((rc = edge_phase(r, cur, Tt, tile, threads, s1, c->s2, c->ev_a))) return rc;
            if (!last && (rc = nccl_exchange(c, edge_xfer(r, Tt), n, c->s2))) return rc;
            if ((rc = interior_phase(r, h, cur, oth, Tt, tile, threads, s1))) return rc;
            cudaEventRecord(c->ev_b, c->s2);
            cudaStreamWaitEvent(s1, c->ev_b, 0);
            if ((rc = assemble_phase(r, (Tt & 1) ? oth : cur, Tt, last, s1))) return rc;
        }
        if (Tt & 1) ci = 1 - ci;
        done += Tt;
    }
    e = cudaMemcpyAsync(d_out_slab, r.row(r.P[ci], off), r.bytes(p.held_hi - p.held_lo), cudaMemcpyDeviceToDevice,
                        s1);
    hhc::set_last_launches(h, r.launches);
    return cuda_rc(e == cudaSuccess ? cudaGetLastError() : e);
}

// `world` virtual ranks of one device, run in lock step through the same
// per-rank phases; the exchange is a device copy from the neighbour's buffer.
extern "C" int stencil_run_dist_local(stencil_t h, int world, const float* d_in, float* d_out, int64_t T,
                                      stencil_tile tile, int threads, int overlap, void* cuda_stream) {
    if (!h || world < 1 || !d_in || !d_out || T < 1 || overlap < 0 || overlap > 1) return STENCIL_EINVAL;
    cudaStream_t s = (cudaStream_t)cuda_stream;
    std::vector<Rank> rk(world);
    auto fail = [&](int rc) {
        cudaStreamSynchronize(s);
        for (auto& r : rk) r.release();
        return rc;
    };
    for (int i = 0; i < world; ++i)
        if (int rc = rk[i].setup(h, i, world, tile.t, overlap != 0)) return fail(rc);
    const size_t nb = rk[0].bytes(tile.t);
    auto exch = [&](const std::vector<Xfer>& xs) {
        for (int i = 0; i < world; ++i) {
            cudaError_t e = cudaSuccess;
            if (xs[i].up_recv) e = cudaMemcpyAsync(xs[i].up_recv, xs[i - 1].dn_send, nb, cudaMemcpyDeviceToDevice, s);
            if (e == cudaSuccess && xs[i].dn_recv)
                e = cudaMemcpyAsync(xs[i].dn_recv, xs[i + 1].up_send, nb, cudaMemcpyDeviceToDevice, s);
            if (e != cudaSuccess) return cuda_rc(e);
        }
        return (int)STENCIL_OK;
    };
    int64_t launches = 0;
    for (auto& r : rk) {
        const Part& p = r.part;
        cudaError_t e = cudaMemcpyAsync(r.row(r.P[0], p.held_lo - p.e0), d_in + p.held_lo * r.inner,
                                        r.bytes(p.held_hi - p.held_lo), cudaMemcpyDeviceToDevice, s);
        if (e != cudaSuccess) return fail(cuda_rc(e));
    }
    int ci = 0;
    int64_t done = 0;
    std::vector<Xfer> xs(world);
    if (rk[0].overlap) {
        for (int i = 0; i < world; ++i) xs[i] = plain_xfer(rk[i], rk[i].P[0]);
        if (int rc = exch(xs)) return fail(rc);
    }
    while (done < T) {
        const int64_t Tt = std::min<int64_t>(tile.t, T - done);
        const bool last = done + Tt >= T;
        int rc;
        for (auto& r : rk)
            if (r.overlap && (rc = edge_phase(r, r.P[ci], Tt, tile, threads, s, s, nullptr))) return fail(rc);
        for (int i = 0; i < world; ++i)
            xs[i] = rk[i].overlap ? (last ? Xfer{} : edge_xfer(rk[i], Tt)) : plain_xfer(rk[i], rk[i].P[ci]);
        if (!rk[0].overlap || !last)
            if ((rc = exch(xs))) return fail(rc);
        for (auto& r : rk) {
            float* cur = r.P[ci];
            float* oth = r.P[1 - ci];
            if (!r.overlap) {
                if ((rc = r.planes(h, r.rows, cur, oth, Tt, tile, threads, s))) return fail(rc);
            } else {
                if ((rc = interior_phase(r, h, cur, oth, Tt, tile, threads, s))) return fail(rc);
                if ((rc = assemble_phase(r, (Tt & 1) ? oth : cur, Tt, last, s))) return fail(rc);
            }
        }
        if (Tt & 1) ci = 1 - ci;
        done += Tt;
    }
    for (auto& r : rk) {
        const Part& p = r.part;
        cudaError_t e = cudaMemcpyAsync(d_out + p.held_lo * r.inner, r.row(r.P[ci], p.held_lo - p.e0),
                                        r.bytes(p.held_hi - p.held_lo), cudaMemcpyDeviceToDevice, s);
        if (e != cudaSuccess) return fail(cuda_rc(e));
        launches += r.launches;
    }
    const int rc = cuda_rc(cudaStreamSynchronize(s));
    for (auto& r : rk) r.release();
    hhc::set_last_launches(h, launches);
    return rc;
}
