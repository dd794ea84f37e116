"""Python binding of libhhc.so (include/hhc.h): argument marshalling only.

Every step of the hot path runs in the library's CUDA kernels; this module
only converts Python/torch arguments to the C ABI.  There is no CPU fallback:
if libhhc.so is missing or no sm_100 device is present, calls raise.

Names follow the C ABI: stencil_create, stencil_run, stencil_run_host,
stencil_run_planes, stencil_destroy, model_predict, model_select_tile,
stencil_tile_resources, stencil_plan_info, stencil_microbench.
"""
from __future__ import annotations

import ctypes
import math
import os
from dataclasses import dataclass

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libhhc.so")

# stencil_kind (include/hhc.h)
JACOBI2D_5PT, HEAT2D_9PT, GRADIENT2D, HEAT3D_7PT, LAPLACIAN3D_27PT, LAPLACIAN2D_5PT = 1, 2, 3, 4, 5, 6
JACOBI1D_3PT = 7          # the paper's 1D derivation case
BINOM1D_R2, BINOM1D_R3, BINOM1D_R4 = 8, 9, 10   # radius-r 1D binomial smoothers
KIND_NAMES = {1: "Jacobi-2D 5-point", 2: "Heat-2D 9-point", 3: "Gradient-2D", 4: "Heat-3D 7-point",
              5: "Laplacian-3D 27-point", 6: "Laplacian-2D 5-point", 7: "Jacobi-1D 3-point",
              8: "Binomial-1D radius 2", 9: "Binomial-1D radius 3", 10: "Binomial-1D radius 4"}
KIND_NDIMS = {1: 2, 2: 2, 3: 2, 4: 3, 5: 3, 6: 2, 7: 1, 8: 1, 9: 1, 10: 1}
KIND_RADIUS = {8: 2, 9: 3, 10: 4}
PLAIN, FUSED = 0, 1
PAPER, EXACT, EXACT_G, EXACT_GW = 0, 1, 2, 3   # EXACT_G: + x-group rows (M9); EXACT_GW: + window rows (M10)

OK, EINVAL, ETILE, ENOMEM, ECUDA, ENCCL, ENODEV = 0, -1, -2, -3, -4, -5, -6


class StencilError(RuntimeError):
    def __init__(self, status: int, what: str = ""):
        super().__init__(f"{what}: {strerror(status)} ({status})")
        self.status = status


class stencil_tile(ctypes.Structure):
    _fields_ = [("t", ctypes.c_int32), ("s1", ctypes.c_int32), ("s2", ctypes.c_int32), ("s3", ctypes.c_int32)]

    def astuple(self):
        return (self.t, self.s1, self.s2, self.s3)

    def __repr__(self):
        return f"stencil_tile{self.astuple()}"


class model_hw_params(ctypes.Structure):
    _fields_ = [("n_sm", ctypes.c_int32), ("n_v", ctypes.c_int32), ("mtb_sm", ctypes.c_int32),
                ("r_sm", ctypes.c_int32), ("m_sm_bytes", ctypes.c_int64), ("m_block_bytes", ctypes.c_int64),
                ("L_s_per_word", ctypes.c_double), ("tau_sync_s", ctypes.c_double),
                ("T_sync_s", ctypes.c_double), ("C_iter_s", ctypes.c_double),
                ("regs_per_thread", ctypes.c_int32), ("geometry", ctypes.c_int32),
                ("threads", ctypes.c_int32), ("max_threads_sm", ctypes.c_int32),
                ("n_gpus", ctypes.c_int32), ("link_bytes_per_s", ctypes.c_double),
                ("link_latency_s", ctypes.c_double), ("dist_overlap", ctypes.c_int32),
                ("window_rows", ctypes.c_double)]


def make_tile(t) -> stencil_tile:
    if isinstance(t, stencil_tile):
        return t
    t = tuple(int(v) for v in t) + (0,) * (4 - len(t))
    return stencil_tile(*t[:4])


def make_hw(**kw) -> model_hw_params:
    hw = model_hw_params()
    for k, v in kw.items():
        setattr(hw, k, v)
    return hw


_lib = None


def load(build_if_missing: bool = False):
    """Load libhhc.so (raises if it is missing: no fallback)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        if build_if_missing:
            from ._build import build
            build()
        else:
            raise ImportError(f"{LIB_PATH} not built; run __graft_entry__.build() "
                              "or python paper_conf_ppopp_prajapatirradg17_b200/_build.py")
    lib = ctypes.CDLL(LIB_PATH)
    P = ctypes.POINTER
    vp = ctypes.c_void_p
    i64p = P(ctypes.c_int64)
    lib.stencil_create.argtypes = [ctypes.c_int, ctypes.c_int, i64p, P(ctypes.c_float), ctypes.c_int,
                                   ctypes.c_int, P(vp)]
    lib.stencil_destroy.argtypes = [vp]
    lib.stencil_destroy.restype = None
    lib.stencil_run.argtypes = [vp, vp, vp, ctypes.c_int64, stencil_tile, ctypes.c_int, vp]
    lib.stencil_run_host.argtypes = [vp, vp, vp, ctypes.c_int64, stencil_tile, ctypes.c_int, vp]
    lib.stencil_run_host_batch.argtypes = [vp, ctypes.c_int, ctypes.POINTER(vp), ctypes.POINTER(vp), ctypes.c_int64,
                                           stencil_tile, ctypes.c_int, vp]
    lib.stencil_run_planes.argtypes = [vp, ctypes.c_int64, vp, vp, ctypes.c_int64, stencil_tile,
                                       ctypes.c_int, vp]
    lib.model_predict.argtypes = [ctypes.c_int, ctypes.c_int, i64p, ctypes.c_int64, stencil_tile,
                                  P(model_hw_params)]
    lib.model_predict.restype = ctypes.c_double
    lib.model_select_tile.argtypes = [ctypes.c_int, ctypes.c_int, i64p, ctypes.c_int64, P(model_hw_params),
                                      ctypes.c_double, P(stencil_tile), P(ctypes.c_int), P(stencil_tile),
                                      ctypes.c_int, P(ctypes.c_int)]
    lib.stencil_tile_resources.argtypes = [ctypes.c_int, ctypes.c_int, stencil_tile, ctypes.c_int, ctypes.c_int,
                                           i64p, P(ctypes.c_int), P(ctypes.c_int)]
    lib.stencil_tile_occupancy.argtypes = [ctypes.c_int, ctypes.c_int, stencil_tile, ctypes.c_int, ctypes.c_int,
                                           P(ctypes.c_int)]
    lib.stencil_plan_info.argtypes = [ctypes.c_int, i64p, ctypes.c_int64, stencil_tile, i64p, i64p, i64p, i64p]
    lib.stencil_microbench.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_int, i64p, ctypes.c_int64,
                                       stencil_tile, ctypes.c_int, P(ctypes.c_double)]
    lib.stencil_strerror.argtypes = [ctypes.c_int]
    lib.stencil_strerror.restype = ctypes.c_char_p
    lib.stencil_profile.argtypes = [vp, vp, vp, ctypes.c_int64, stencil_tile, ctypes.c_int, vp,
                                    P(ctypes.c_double), P(ctypes.c_int64)]
    lib.stencil_last_launches.argtypes = [vp]
    lib.stencil_last_launches.restype = ctypes.c_int64
    lib.stencil_run_wavefront.argtypes = [vp, vp, vp, ctypes.c_int64, stencil_tile, vp]
    lib.stencil_wavefront_info.argtypes = [i64p, ctypes.c_int64, stencil_tile, i64p, i64p, i64p]
    lib.model_predict_wavefront.argtypes = [ctypes.c_int, ctypes.c_int, i64p, ctypes.c_int64, stencil_tile,
                                            P(model_hw_params)]
    lib.model_predict_wavefront.restype = ctypes.c_double
    lib.model_select_wavefront_tile.argtypes = [ctypes.c_int, ctypes.c_int, i64p, ctypes.c_int64,
                                                P(model_hw_params), ctypes.c_double, P(stencil_tile),
                                                P(stencil_tile), ctypes.c_int, P(ctypes.c_int)]
    lib.stencil_dist_get_unique_id.argtypes = [ctypes.c_char_p]
    lib.stencil_dist_init.argtypes = [ctypes.c_char_p, ctypes.c_int, ctypes.c_int, ctypes.c_int, P(vp)]
    lib.stencil_dist_set_overlap.argtypes = [vp, ctypes.c_int]
    lib.stencil_dist_destroy.argtypes = [vp]
    lib.stencil_dist_destroy.restype = None
    lib.stencil_dist_partition.argtypes = [ctypes.c_int64, ctypes.c_int, ctypes.c_int, ctypes.c_int64, i64p]
    lib.stencil_run_dist.argtypes = [vp, vp, vp, vp, ctypes.c_int64, stencil_tile, ctypes.c_int, vp]
    lib.stencil_run_dist_local.argtypes = [vp, ctypes.c_int, vp, vp, ctypes.c_int64, stencil_tile, ctypes.c_int,
                                           ctypes.c_int, vp]
    lib.stencil_hexdist_partition.argtypes = [ctypes.c_int64, ctypes.c_int, ctypes.c_int, stencil_tile, i64p]
    lib.stencil_run_hexdist_local.argtypes = [vp, ctypes.c_int, vp, vp, ctypes.c_int64, stencil_tile, ctypes.c_int,
                                              vp]
    lib.stencil_hexdist_create.argtypes = [vp, ctypes.c_int, ctypes.c_int, stencil_tile, ctypes.c_char_p, P(vp)]
    lib.stencil_hexdist_connect.argtypes = [vp, vp, ctypes.c_char_p, ctypes.c_char_p]
    lib.stencil_run_hexdist.argtypes = [vp, vp, vp, vp, ctypes.c_int64, ctypes.c_int, vp]
    lib.stencil_hexdist_destroy.argtypes = [vp]
    lib.stencil_hexdist_destroy.restype = None
    _lib = lib
    return lib


def strerror(status: int) -> str:
    try:
        return load().stencil_strerror(int(status)).decode()
    except ImportError:
        return str(status)


def _check(rc: int, what: str):
    if rc != 0:
        raise StencilError(rc, what)


def _dims(dims):
    d = [int(x) for x in dims]
    return (ctypes.c_int64 * len(d))(*d), len(d)


def _ptr(x) -> int:
    """Device/host pointer of a torch tensor (or an int)."""
    if isinstance(x, int):
        return x
    if hasattr(x, "data_ptr"):
        if not x.is_contiguous() or str(x.dtype) != "torch.float32":
            raise ValueError("tensors must be contiguous float32")
        return x.data_ptr()
    if hasattr(x, "ctypes"):
        return x.ctypes.data
    raise TypeError(type(x))


def _stream(stream) -> int:
    if stream is None:
        import torch
        return torch.cuda.current_stream().cuda_stream
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


@dataclass
class Stencil:
    """Owning wrapper around a stencil_t handle."""
    handle: int
    kind: int
    dims: tuple
    mode: int

    def __del__(self):
        try:
            stencil_destroy(self)
        except Exception:
            pass


def stencil_create(kind: int, dims, coeffs=None, mode: int = FUSED) -> Stencil:
    lib = load()
    d, nd = _dims(dims)
    h = ctypes.c_void_p()
    if coeffs is None:
        cp, nc = None, 0
    else:
        arr = (ctypes.c_float * len(coeffs))(*[float(c) for c in coeffs])
        cp, nc = arr, len(coeffs)
    _check(lib.stencil_create(int(kind), nd, d, cp, nc, int(mode), ctypes.byref(h)), "stencil_create")
    return Stencil(h.value, int(kind), tuple(int(x) for x in dims), int(mode))


def stencil_destroy(s: Stencil):
    if s is not None and s.handle:
        load().stencil_destroy(s.handle)
        s.handle = 0


def stencil_run(s: Stencil, d_in, d_out, T: int, tile, threads: int = 0, stream=None):
    _check(load().stencil_run(s.handle, _ptr(d_in), _ptr(d_out), int(T), make_tile(tile), int(threads),
                              _stream(stream)), "stencil_run")


def stencil_run_host(s: Stencil, h_in, h_out, T: int, tile, threads: int = 0, stream=None):
    _check(load().stencil_run_host(s.handle, _ptr(h_in), _ptr(h_out), int(T), make_tile(tile), int(threads),
                                   _stream(stream)), "stencil_run_host")


def stencil_run_host_batch(s: Stencil, h_ins, h_outs, T: int, tile, threads: int = 0, stream=None):
    """n problems host -> device -> host with the copies overlapping the runs (the C call)."""
    n = len(h_ins)
    if n != len(h_outs) or n < 1:
        raise ValueError("stencil_run_host_batch: h_ins and h_outs must have the same non-zero length")
    ins = (ctypes.c_void_p * n)(*[_ptr(x) for x in h_ins])
    outs = (ctypes.c_void_p * n)(*[_ptr(x) for x in h_outs])
    _check(load().stencil_run_host_batch(s.handle, n, ins, outs, int(T), make_tile(tile), int(threads),
                                         _stream(stream)), "stencil_run_host_batch")


def stencil_run_planes(s: Stencil, rows: int, plane0, plane1, T: int, tile, threads: int = 0, stream=None):
    _check(load().stencil_run_planes(s.handle, int(rows), _ptr(plane0), _ptr(plane1), int(T), make_tile(tile),
                                     int(threads), _stream(stream)), "stencil_run_planes")


def stencil_profile(s: Stencil, d_in, d_out, T: int, tile, threads: int = 0, stream=None):
    """(summed device seconds of the HHC kernel launches, number of launches)."""
    sec = ctypes.c_double()
    n = ctypes.c_int64()
    _check(load().stencil_profile(s.handle, _ptr(d_in), _ptr(d_out), int(T), make_tile(tile), int(threads),
                                  _stream(stream), ctypes.byref(sec), ctypes.byref(n)), "stencil_profile")
    return sec.value, n.value


def stencil_run_wavefront(s: Stencil, d_in, d_out, T: int, tile, stream=None):
    """Wavefront-parallel Jacobi-1D (hhc.h): tile = (t, s1) parallelogram."""
    _check(load().stencil_run_wavefront(s.handle, _ptr(d_in), _ptr(d_out), int(T), make_tile(tile),
                                        _stream(stream)), "stencil_run_wavefront")


def stencil_wavefront_info(dims, T: int, tile):
    """(wavefronts = launches, tiles in total, tiles of the widest wavefront)."""
    d, _ = _dims(dims)
    out = [ctypes.c_int64() for _ in range(3)]
    _check(load().stencil_wavefront_info(d, int(T), make_tile(tile), *[ctypes.byref(o) for o in out]),
           "stencil_wavefront_info")
    return tuple(o.value for o in out)


def model_predict_wavefront(dims, T: int, tile, hw: model_hw_params) -> float:
    d, nd = _dims(dims)
    return float(load().model_predict_wavefront(JACOBI1D_3PT, nd, d, int(T), make_tile(tile), ctypes.byref(hw)))


def model_select_wavefront_tile(dims, T: int, hw: model_hw_params, within: float = 0.10, cap: int = 10000):
    """(best (t, s1), candidate (t, s1) list) for the wavefront schedule."""
    d, nd = _dims(dims)
    best = stencil_tile()
    cands = (stencil_tile * cap)()
    n = ctypes.c_int()
    _check(load().model_select_wavefront_tile(JACOBI1D_3PT, nd, d, int(T), ctypes.byref(hw), float(within),
                                              ctypes.byref(best), cands, cap, ctypes.byref(n)),
           "model_select_wavefront_tile")
    return best.astuple()[:2], [cands[i].astuple()[:2] for i in range(min(n.value, cap))]


def stencil_last_launches(s: Stencil) -> int:
    return int(load().stencil_last_launches(s.handle))


def model_predict(kind: int, dims, T: int, tile, hw: model_hw_params) -> float:
    d, nd = _dims(dims)
    return float(load().model_predict(int(kind), nd, d, int(T), make_tile(tile), ctypes.byref(hw)))


def model_select_tile(kind: int, dims, T: int, hw: model_hw_params, within: float = 0.10, cap: int = 100000):
    """Returns (best tile tuple, best threads, list of candidate tile tuples)."""
    d, nd = _dims(dims)
    best = stencil_tile()
    thr = ctypes.c_int()
    cands = (stencil_tile * cap)()
    n = ctypes.c_int()
    _check(load().model_select_tile(int(kind), nd, d, int(T), ctypes.byref(hw), float(within),
                                    ctypes.byref(best), ctypes.byref(thr), cands, cap, ctypes.byref(n)),
           "model_select_tile")
    return best.astuple(), thr.value, [cands[i].astuple() for i in range(min(n.value, cap))]


def stencil_tile_resources(ndims: int, tile, threads: int = 0, kind: int = 0, mode: int = FUSED):
    """(smem bytes, threads per block, registers per thread) of the kernel the
    library launches; registers are 0 for kind = 0 or without a CUDA device."""
    sm = ctypes.c_int64()
    thr = ctypes.c_int()
    regs = ctypes.c_int()
    _check(load().stencil_tile_resources(int(kind), int(ndims), make_tile(tile), int(threads), int(mode),
                                         ctypes.byref(sm), ctypes.byref(thr), ctypes.byref(regs)),
           "stencil_tile_resources")
    return sm.value, thr.value, regs.value


def stencil_tile_occupancy(kind: int, tile, threads: int = 0, mode: int = FUSED) -> int:
    """Resident blocks per SM of the kernel for (kind, tile, threads) (CUDA occupancy API)."""
    k = ctypes.c_int()
    _check(load().stencil_tile_occupancy(int(kind), KIND_NDIMS[int(kind)], make_tile(tile), int(threads), int(mode),
                                         ctypes.byref(k)), "stencil_tile_occupancy")
    return k.value


def stencil_dist_get_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(128)
    _check(load().stencil_dist_get_unique_id(buf), "stencil_dist_get_unique_id")
    return buf.raw


def stencil_dist_init(uid, rank: int, world: int, device: int):
    """NCCL communicator of this rank (opaque); uid = rank 0's stencil_dist_get_unique_id()."""
    comm = ctypes.c_void_p()
    _check(load().stencil_dist_init(uid if uid else None, int(rank), int(world), int(device), ctypes.byref(comm)),
           "stencil_dist_init")
    return comm


def stencil_dist_set_overlap(comm, overlap: int):
    _check(load().stencil_dist_set_overlap(comm, int(overlap)), "stencil_dist_set_overlap")


def stencil_dist_destroy(comm):
    load().stencil_dist_destroy(comm)


def stencil_dist_partition(S1: int, rank: int, world: int, g: int):
    """(r0, r1, e0, e1, held_lo, held_hi) of one rank's slab (host only)."""
    out = (ctypes.c_int64 * 6)()
    _check(load().stencil_dist_partition(int(S1), int(rank), int(world), int(g), out), "stencil_dist_partition")
    return tuple(out)


def stencil_run_dist(h, comm, d_in_slab, d_out_slab, T: int, tile, threads: int = 0, stream=None):
    _check(load().stencil_run_dist(h.handle, comm, _ptr(d_in_slab), _ptr(d_out_slab), int(T), make_tile(tile),
                                   int(threads), _stream(stream)), "stencil_run_dist")


def stencil_run_dist_local(h, world: int, d_in, d_out, T: int, tile, threads: int = 0, overlap: int = 0,
                           stream=None):
    _check(load().stencil_run_dist_local(h.handle, int(world), _ptr(d_in), _ptr(d_out), int(T), make_tile(tile),
                                         int(threads), int(overlap), _stream(stream)), "stencil_run_dist_local")


def stencil_hexdist_partition(S1: int, rank: int, world: int, tile):
    """f1: (b0, b1, x_lo, x_hi, held_lo, held_hi) of one rank (host only)."""
    out = (ctypes.c_int64 * 6)()
    _check(load().stencil_hexdist_partition(int(S1), int(rank), int(world), make_tile(tile), out),
           "stencil_hexdist_partition")
    return tuple(out)


def stencil_run_hexdist_local(h, world: int, d_in, d_out, T: int, tile, threads: int = 0, stream=None):
    _check(load().stencil_run_hexdist_local(h.handle, int(world), _ptr(d_in), _ptr(d_out), int(T), make_tile(tile),
                                            int(threads), _stream(stream)), "stencil_run_hexdist_local")


def stencil_hexdist_create(h, rank: int, world: int, tile):
    """f1 across processes: (opaque object, 192 bytes of IPC handles to give the neighbours)."""
    buf = ctypes.create_string_buffer(192)
    obj = ctypes.c_void_p()
    _check(load().stencil_hexdist_create(h.handle, int(rank), int(world), make_tile(tile), buf, ctypes.byref(obj)),
           "stencil_hexdist_create")
    return obj, buf.raw


def stencil_hexdist_connect(h, obj, lo: bytes | None, hi: bytes | None):
    _check(load().stencil_hexdist_connect(h.handle, obj, lo, hi), "stencil_hexdist_connect")


def stencil_run_hexdist(h, obj, d_in_stored, d_out_slab, T: int, threads: int = 0, stream=None):
    _check(load().stencil_run_hexdist(h.handle, obj, _ptr(d_in_stored), _ptr(d_out_slab), int(T), int(threads),
                                      _stream(stream)), "stencil_run_hexdist")


def stencil_hexdist_destroy(obj):
    load().stencil_hexdist_destroy(obj)


def stencil_plan_info(dims, T: int, tile):
    d, nd = _dims(dims)
    out = [ctypes.c_int64() for _ in range(4)]
    _check(load().stencil_plan_info(nd, d, int(T), make_tile(tile), *[ctypes.byref(o) for o in out]),
           "stencil_plan_info")
    return tuple(o.value for o in out)


def stencil_microbench(which: int, kind: int = HEAT2D_9PT, dims=(3, 3), T: int = 1, tile=(2, 1, 32, 0),
                       threads: int = 0) -> float:
    d, nd = _dims(dims)
    v = ctypes.c_double()
    _check(load().stencil_microbench(int(which), int(kind), nd, d, int(T), make_tile(tile), int(threads),
                                     ctypes.byref(v)), "stencil_microbench")
    return v.value


def updates(dims, T: int, kind: int = 0) -> int:
    """Interior stencil updates of a run: T * prod(S_d - 2R) (ring width R = 1,
    2-4 for the f4 kinds)."""
    R = KIND_RADIUS.get(int(kind), 1)
    return int(T) * math.prod(int(x) - 2 * R for x in dims)


EXPORTED_SYMBOLS = ["stencil_create", "stencil_destroy", "stencil_run", "stencil_run_host", "stencil_run_host_batch",
                    "stencil_run_planes", "model_predict", "model_select_tile", "stencil_tile_resources", "stencil_tile_occupancy",
                    "stencil_plan_info", "stencil_microbench", "stencil_strerror", "stencil_last_launches",
                    "stencil_profile", "stencil_run_wavefront", "stencil_wavefront_info",
                    "model_predict_wavefront", "model_select_wavefront_tile", "stencil_dist_get_unique_id",
                    "stencil_dist_init", "stencil_dist_set_overlap", "stencil_dist_destroy", "stencil_dist_partition",
                    "stencil_run_dist", "stencil_run_dist_local", "stencil_hexdist_partition",
                    "stencil_run_hexdist_local", "stencil_hexdist_create", "stencil_hexdist_connect",
                    "stencil_run_hexdist", "stencil_hexdist_destroy"]
