"""Python binding of the B200-native LoRAStencil engine (liblora_stencil.so, include/lora_stencil.h).

Argument marshalling only: every step of the stencil runs in the CUDA kernels of the shared
library.  There is no CPU fallback — importing this package fails loudly if the library is
missing, and the run calls require device pointers (torch CUDA tensors) or, for
``lora_stencil_run_host``, host buffers that the library itself copies to the GPU.

The function names are the C-ABI names.  ``Stencil`` is a thin convenience wrapper.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("LORA_LIB", os.path.join(_PKG, "liblora_stencil.so"))  # override: variant builds

if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} is missing: build it with `python -c 'import __graft_entry__ as g; g.build()'` "
                      "(there is no CPU fallback)")
_lib = ctypes.CDLL(LIB_PATH)

LORA_OK = 0
LORA_ERR_INVALID_ARG = -1
LORA_ERR_UNSUPPORTED = -2
LORA_ERR_ALIAS = -3
LORA_ERR_CUDA = -4
LORA_ERR_NCCL = -5
LORA_ERR_OOM = -6
LORA_ERR_FACTOR = -7

LORA_ENGINE_AUTO = 0
LORA_ENGINE_TC = 1
LORA_ENGINE_RDG_CUDA = 2
LORA_ENGINE_DIRECT = 3
ENGINES = {"auto": 0, "tc": 1, "rdg_cuda": 2, "direct": 3}
ENGINE_NAMES = {v: k for k, v in ENGINES.items()}


class lora_plan_opts(ctypes.Structure):
    _fields_ = [("engine", ctypes.c_int), ("fuse_k", ctypes.c_int), ("reserved", ctypes.c_int * 6)]


class lora_plan_info(ctypes.Structure):
    _fields_ = [("ndim", ctypes.c_int), ("radius", ctypes.c_int), ("grid", ctypes.c_int64 * 3),
                ("engine", ctypes.c_int), ("n_terms", ctypes.c_int), ("n_tc_chain", ctypes.c_int),
                ("n_tc_single", ctypes.c_int), ("n_cuda", ctypes.c_int), ("n_planes_pointwise", ctypes.c_int),
                ("z_symmetric", ctypes.c_int), ("fuse_k", ctypes.c_int), ("halo_depth", ctypes.c_int),
                ("tile_m", ctypes.c_int), ("tile_n", ctypes.c_int), ("single_launch", ctypes.c_int),
                ("recon_err", ctypes.c_double),
                ("growth", ctypes.c_double), ("fma_per_point_issued", ctypes.c_double),
                ("fma_per_point_direct", ctypes.c_double), ("fma_per_point_separable", ctypes.c_double),
                ("paper_points_per_update", ctypes.c_int), ("paper_rdg_frag_per_point", ctypes.c_double),
                ("paper_convstencil_frag_per_point", ctypes.c_double), ("paper_convstencil_over_rdg", ctypes.c_double),
                ("paper_mma_per_point", ctypes.c_double), ("paper_convstencil_mma_per_point", ctypes.c_double),
                ("paper_fragment_waste", ctypes.c_int)]

    def as_dict(self):
        d = {f: getattr(self, f) for f, _ in self._fields_}
        d["grid"] = list(self.grid)
        d["engine_name"] = ENGINE_NAMES.get(self.engine, "?")
        return d


_P = ctypes.c_void_p
_sig = {
    "lora_stencil_plan": (_P, [_P, ctypes.c_int, ctypes.c_int, _P]),
    "lora_stencil_plan_ex": (_P, [_P, ctypes.c_int, ctypes.c_int, _P, _P]),
    "lora_stencil_run": (ctypes.c_int, [_P, _P, _P, ctypes.c_int64, _P]),
    "lora_stencil_run_host": (ctypes.c_int, [_P, _P, _P, ctypes.c_int64, _P]),
    "lora_stencil_run_host_async": (ctypes.c_int, [_P, _P, _P, ctypes.c_int64, _P]),
    "lora_stencil_plan_query": (ctypes.c_int, [_P, _P]),
    "lora_stencil_plan_terms": (ctypes.c_int, [_P, ctypes.c_int, _P, _P, _P, _P, _P, _P]),
    "lora_stencil_plan_destroy": (None, [_P]),
    "lora_stencil_comm_id_size": (ctypes.c_size_t, []),
    "lora_stencil_comm_get_id": (ctypes.c_int, [_P]),
    "lora_stencil_comm_init": (ctypes.c_int, [_P, ctypes.c_int, ctypes.c_int, _P]),
    "lora_stencil_run_dist": (ctypes.c_int, [_P, _P, _P, _P, ctypes.c_int64, _P]),
    "lora_stencil_comm_destroy": (None, [_P]),
    "lora_stencil_dist_exchange_plan": (ctypes.c_int, [_P, ctypes.c_int, ctypes.c_int, _P, _P, _P, _P]),
    "lora_stencil_dist_exchange_plan_ex": (ctypes.c_int, [_P, ctypes.c_int, ctypes.c_int, ctypes.c_int64, _P, _P, _P, _P]),
    "lora_stencil_p2p_create": (ctypes.c_int, [_P, _P, ctypes.c_int, ctypes.c_int]),
    "lora_stencil_p2p_handle_size": (ctypes.c_size_t, []),
    "lora_stencil_p2p_get_handle": (ctypes.c_int, [_P, _P]),
    "lora_stencil_p2p_connect": (ctypes.c_int, [_P, _P, _P]),
    "lora_stencil_p2p_connect_local": (ctypes.c_int, [_P, _P, _P]),
    "lora_stencil_p2p_buffer": (_P, [_P, ctypes.c_int]),
    "lora_stencil_p2p_view": (_P, [_P, ctypes.c_int]),
    "lora_stencil_run_dist_p2p": (ctypes.c_int, [_P, _P, _P, _P, ctypes.c_int64, _P]),
    "lora_stencil_p2p_status": (ctypes.c_int, [_P]),
    "lora_stencil_p2p_destroy": (None, [_P]),
    "lora_stencil_last_error": (ctypes.c_char_p, []),
    "lora_stencil_last_status": (ctypes.c_int, []),
    "lora_stencil_version": (ctypes.c_char_p, []),
}
for _name, (_res, _args) in _sig.items():
    _f = getattr(_lib, _name)
    _f.restype = _res
    _f.argtypes = _args

EXPORTED = tuple(_sig)


class LoraError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__(f"lora_stencil error {code}: {msg}")
        self.code = code


def lora_stencil_last_error() -> str:
    return _lib.lora_stencil_last_error().decode()


def lora_stencil_version() -> str:
    return _lib.lora_stencil_version().decode()


def _check(rc):
    if rc != LORA_OK:
        raise LoraError(rc, lora_stencil_last_error())
    return rc


def lora_stencil_plan_ex(weights, ndim: int, radius: int, grid_shape, engine=0, fuse_k: int = 0):
    """Host-only planning (no CUDA call).  Returns an opaque plan handle (int)."""
    w = np.ascontiguousarray(weights, dtype=np.float64)
    g = np.ascontiguousarray(grid_shape, dtype=np.int64)
    if isinstance(engine, str):
        engine = ENGINES[engine]
    opts = lora_plan_opts(engine=int(engine), fuse_k=int(fuse_k))
    h = _lib.lora_stencil_plan_ex(w.ctypes.data, int(ndim), int(radius), g.ctypes.data, ctypes.byref(opts))
    if not h:
        raise LoraError(int(_lib.lora_stencil_last_status()), lora_stencil_last_error())
    return h


def lora_stencil_plan(weights, ndim: int, radius: int, grid_shape):
    return lora_stencil_plan_ex(weights, ndim, radius, grid_shape)


def lora_stencil_plan_destroy(plan) -> None:
    _lib.lora_stencil_plan_destroy(plan)


def lora_stencil_plan_query(plan) -> dict:
    info = lora_plan_info()
    _check(_lib.lora_stencil_plan_query(plan, ctypes.byref(info)))
    return info.as_dict()


def _padded_elems(plan) -> int:
    info = lora_stencil_plan_query(plan)
    n = 1
    for i in range(info["ndim"]):
        n *= int(info["grid"][i]) + 2 * int(info["radius"])
    return n


def _host_ptr(a, plan, what: str) -> int:
    """Pointer of a host buffer after checking that it is what the C side will copy: float64,
    C-contiguous, exactly the plan's padded element count (prod(N_i + 2r))."""
    n = _padded_elems(plan)
    if isinstance(a, np.ndarray):
        ok = a.dtype == np.float64 and a.flags["C_CONTIGUOUS"] and a.size == n
        ptr = a.ctypes.data
    else:  # torch CPU tensor
        ok = (not a.is_cuda) and a.dtype.is_floating_point and a.element_size() == 8 and a.is_contiguous() \
            and a.numel() == n
        ptr = a.data_ptr()
    if not ok:
        raise ValueError(f"{what}: expected a C-contiguous float64 host buffer of {n} elements (the plan's padded shape)")
    return ptr


def lora_stencil_plan_terms(plan, radius: int | None = None):
    """The plan's rank-1 terms.  The term length is taken from the plan itself (2r+1 with the
    plan's radius); `radius`, if given, must match it."""
    r = int(lora_stencil_plan_query(plan)["radius"])
    if radius is not None and int(radius) != r:
        raise ValueError(f"radius {radius} does not match the plan's radius {r}")
    n = ctypes.c_int(0)
    _check(_lib.lora_stencil_plan_terms(plan, 0, ctypes.byref(n), None, None, None, None, None))
    k, m = n.value, 2 * r + 1
    plane = np.zeros(k, np.int32); kind = np.zeros(k, np.int32); rad = np.zeros(k, np.int32)
    u = np.zeros((k, m)); v = np.zeros((k, m))
    if k:
        _check(_lib.lora_stencil_plan_terms(plan, k, ctypes.byref(n), plane.ctypes.data, kind.ctypes.data,
                                            rad.ctypes.data, u.ctypes.data, v.ctypes.data))
    return [dict(plane=int(plane[i]), kind=int(kind[i]), radius=int(rad[i]), u=u[i], v=v[i]) for i in range(k)]


def lora_stencil_run(plan, in_ptr: int, out_ptr: int, timesteps: int, stream: int = 0) -> None:
    """Device pointers (e.g. tensor.data_ptr()), cudaStream_t as int (0 = legacy default)."""
    _check(_lib.lora_stencil_run(plan, in_ptr, out_ptr, int(timesteps), stream or None))


def lora_stencil_run_host(plan, in_host: np.ndarray, out_host: np.ndarray, timesteps: int, stream: int = 0) -> None:
    """Host buffers (numpy arrays or torch CPU tensors, ideally pinned); synchronous."""
    ip = _host_ptr(in_host, plan, "in_host")
    op = _host_ptr(out_host, plan, "out_host")
    _check(_lib.lora_stencil_run_host(plan, ip, op, int(timesteps), stream or None))


def lora_stencil_run_host_async(plan, in_host, out_host, timesteps: int, stream: int) -> None:
    """Host buffers (pinned); enqueued on `stream` (not 0), the caller synchronises it."""
    ip = _host_ptr(in_host, plan, "in_host")
    op = _host_ptr(out_host, plan, "out_host")
    _check(_lib.lora_stencil_run_host_async(plan, ip, op, int(timesteps), stream or None))


def lora_stencil_comm_id_size() -> int:
    return int(_lib.lora_stencil_comm_id_size())


def lora_stencil_comm_get_id() -> bytes:
    buf = ctypes.create_string_buffer(lora_stencil_comm_id_size())
    _check(_lib.lora_stencil_comm_get_id(buf))
    return buf.raw


def lora_stencil_comm_init(nranks: int, rank: int, uid: bytes):
    c = ctypes.c_void_p(0)
    buf = ctypes.create_string_buffer(uid, len(uid))
    _check(_lib.lora_stencil_comm_init(ctypes.byref(c), int(nranks), int(rank), buf))
    return c.value


def lora_stencil_run_dist(plan, comm, in_ptr: int, out_ptr: int, timesteps: int, stream: int = 0) -> None:
    _check(_lib.lora_stencil_run_dist(plan, comm, in_ptr, out_ptr, int(timesteps), stream or None))


def lora_stencil_comm_destroy(comm) -> None:
    _lib.lora_stencil_comm_destroy(comm)


def lora_stencil_p2p_create(plan, nranks: int, rank: int):
    """Device-initiated halo exchange endpoint for `plan` (local slab) on the current device."""
    c = ctypes.c_void_p(0)
    _check(_lib.lora_stencil_p2p_create(ctypes.byref(c), plan, int(nranks), int(rank)))
    return c.value


def lora_stencil_p2p_handle_size() -> int:
    return int(_lib.lora_stencil_p2p_handle_size())


def lora_stencil_p2p_get_handle(c) -> bytes:
    buf = ctypes.create_string_buffer(lora_stencil_p2p_handle_size())
    _check(_lib.lora_stencil_p2p_get_handle(c, buf))
    return buf.raw


def lora_stencil_p2p_connect(c, lo_handle, hi_handle) -> None:
    """Other-process neighbours: their handles (bytes) or None where there is no neighbour."""
    lo = ctypes.create_string_buffer(lo_handle, len(lo_handle)) if lo_handle is not None else None
    hi = ctypes.create_string_buffer(hi_handle, len(hi_handle)) if hi_handle is not None else None
    _check(_lib.lora_stencil_p2p_connect(c, lo, hi))


def lora_stencil_p2p_connect_local(c, lo, hi) -> None:
    """Same-process neighbours (endpoint handles or None)."""
    _check(_lib.lora_stencil_p2p_connect_local(c, lo, hi))


def lora_stencil_p2p_buffer(c, i: int) -> int:
    return int(_lib.lora_stencil_p2p_buffer(c, int(i)) or 0)


def lora_stencil_p2p_view(c, i: int) -> int:
    """Caller-layout view (padded local slab, R-deep halos) inside exchange buffer i: pass view 0 as
    `in` and view (launches % 2) as `out` of lora_stencil_run_dist_p2p to skip the copies."""
    return int(_lib.lora_stencil_p2p_view(c, int(i)) or 0)


def lora_stencil_run_dist_p2p(plan, c, in_ptr: int, out_ptr: int, timesteps: int, stream: int = 0) -> None:
    _check(_lib.lora_stencil_run_dist_p2p(plan, c, in_ptr, out_ptr, int(timesteps), stream or None))


def lora_stencil_p2p_status(c) -> None:
    _check(_lib.lora_stencil_p2p_status(c))


def lora_stencil_p2p_destroy(c) -> None:
    _lib.lora_stencil_p2p_destroy(c)


def lora_stencil_dist_exchange_plan(plan, rank: int, nranks: int, halo_depth: int | None = None):
    """[(kind 'send'|'recv', peer, element offset, element count)] in NCCL-group issue order; with
    halo_depth, the plan for a deep-halo slab buffer (lora_stencil_dist_exchange_plan_ex)."""
    a = [np.zeros(4, np.int64) for _ in range(4)]
    if halo_depth is None:
        m = _lib.lora_stencil_dist_exchange_plan(plan, int(rank), int(nranks), *[x.ctypes.data for x in a])
    else:
        m = _lib.lora_stencil_dist_exchange_plan_ex(plan, int(rank), int(nranks), int(halo_depth),
                                                    *[x.ctypes.data for x in a])
    if m < 0:
        raise LoraError(m, lora_stencil_last_error())
    return [("send" if a[0][i] == 0 else "recv", int(a[1][i]), int(a[2][i]), int(a[3][i])) for i in range(m)]


class Stencil:
    """Owns a plan.  ``run(x_in, x_out, T)`` on torch CUDA tensors (padded, float64, contiguous)."""

    def __init__(self, weights, grid_shape, engine="auto", fuse_k: int = 0):
        w = np.asarray(weights, dtype=np.float64)
        self.ndim = w.ndim
        self.radius = (w.shape[0] - 1) // 2
        self.grid_shape = tuple(int(x) for x in grid_shape)
        self.padded_shape = tuple(n + 2 * self.radius for n in self.grid_shape)
        self.plan = lora_stencil_plan_ex(w, self.ndim, self.radius, self.grid_shape, engine, fuse_k)

    def info(self) -> dict:
        return lora_stencil_plan_query(self.plan)

    def terms(self):
        return lora_stencil_plan_terms(self.plan)

    def run(self, x_in, x_out, timesteps: int, stream=None) -> None:
        for x in (x_in, x_out):
            if not x.is_cuda or x.dtype.itemsize != 8 or not x.is_contiguous() or tuple(x.shape) != self.padded_shape:
                raise ValueError(f"expected contiguous float64 CUDA tensors of shape {self.padded_shape}")
        s = stream.cuda_stream if stream is not None else 0
        if s == 0:
            import torch
            s = torch.cuda.current_stream(x_in.device).cuda_stream
        lora_stencil_run(self.plan, x_in.data_ptr(), x_out.data_ptr(), timesteps, s)

    def run_host(self, a_in, a_out, timesteps: int, stream: int = 0) -> None:
        for a in (a_in, a_out):
            if tuple(a.shape) != self.padded_shape:
                raise ValueError(f"expected host arrays of shape {self.padded_shape}")
        lora_stencil_run_host(self.plan, a_in, a_out, timesteps, stream)

    def close(self):
        if self.plan:
            lora_stencil_plan_destroy(self.plan)
            self.plan = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
