"""Thin ctypes binding over ``libctaclust.so`` (include/ctaclust.h).

Argument marshalling only: every step of the hot path runs in the library's
sm_100a kernels.  Names follow the C ABI (``cc_plan_create`` -> :class:`Plan`,
``cc_launch`` -> :func:`launch` and the per-kernel helpers).  Device buffers are
passed as torch CUDA tensors (PyTorch is used for memory and streams only).
A missing library raises :class:`CtaclustError`; there is no fallback.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
# CTACLUST_LIB: an alternative build of the same library (diagnostic builds
# with CC_DEFS, scripts/); still the CUDA library, never a fallback
LIB_PATH = os.environ.get("CTACLUST_LIB") or os.path.join(_HERE, "libctaclust.so")

# ---- enums (ctaclust.h) ----------------------------------------------------
ORDER_ROW, ORDER_COL, ORDER_TILE, ORDER_USER = 0, 1, 2, 3
ORDERS = {"row": ORDER_ROW, "col": ORDER_COL, "tile": ORDER_TILE, "user": ORDER_USER}
BACKEND_DEFAULT, BACKEND_AGENT, BACKEND_TBCLUSTER, BACKEND_AGENT_IDENTITY, BACKEND_REDIRECT, BACKEND_AGENT_STATIC = 0, 1, 2, 3, 4, 5
BACKENDS = {"default": 0, "agent": 1, "tbcluster": 2, "identity": 3, "redirect": 4, "static": 5}
K_CENSUS, K_MATVEC, K_ATAX, K_BICG, K_MVT, K_JACOBI5, K_CONV2D, K_SPMV = range(8)
STAGINGS = {"default": 0, "tma": 1, "l1": 2, "direct": 3}
KERNELS = {"census": 0, "matvec": 1, "atax": 2, "bicg": 3, "mvt": 4, "jacobi5": 5, "conv2d": 6, "spmv": 7,
           "hist64": 8, "jacobi5_halo": 9, "atax_fused": 10, "spmv_shub": 11,
           "jacobi5_wave": 12}
SPMV_SHUB_SLOTS = 8192     # include/ctaclust.h CC_SPMV_SHUB_SLOTS (shared-memory hub tier)
STATUS = {0: "CC_OK", -1: "CC_ERR_INVALID_ARG", -2: "CC_ERR_OVERFLOW", -3: "CC_ERR_NOT_PERMUTATION",
          -4: "CC_ERR_CUDA", -5: "CC_ERR_NCCL", -6: "CC_ERR_UNSUPPORTED", -7: "CC_ERR_NO_DEVICE",
          -8: "CC_ERR_BUSY"}

# every symbol include/ctaclust.h declares (checked by tests/test_abi.py)
EXPORTS = ["cc_plan_create", "cc_plan_destroy", "cc_plan_info", "cc_plan_table", "cc_plan_lookup",
           "cc_plan_invert", "cc_device_info", "cc_sm_rank_table", "cc_launch_opts_default",
           "cc_kernel_grid", "cc_max_agents", "cc_launch", "cc_spmv_partition", "cc_spmv_inspect", "cc_l1_reuse_probe", "cc_comm_unique_id",
           "cc_comm_init", "cc_comm_destroy", "cc_halo_exchange", "cc_allreduce_sum", "cc_allgather",
           "cc_peer_access", "cc_l2_persist", "cc_ipc_handle", "cc_ipc_open", "cc_ipc_close", "cc_status_string", "cc_last_error", "cc_last_cuda_error", "cc_version"]


class CtaclustError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status


# ---- structs ----------------------------------------------------------------
_i32, _i64, _vp = ctypes.c_int32, ctypes.c_int64, ctypes.c_void_p


class PlanDesc(ctypes.Structure):
    _fields_ = [("gx", _i32), ("gy", _i32), ("order", _i32), ("tile_w", _i32), ("tile_h", _i32),
                ("num_clusters", _i32), ("user_order", _vp), ("device", _i32)]


class LaunchOpts(ctypes.Structure):
    _fields_ = [("backend", _i32), ("active_agents", _i32), ("max_agents", _i32), ("stages", _i32),
                ("batch", _i32), ("staging", _i32), ("steal", _i32), ("cluster_size", _i32), ("d_census", _vp),
                ("d_exec_sm", _vp),
                ("d_map", _vp), ("l2_hint", _i32), ("carveout", _i32)]


class CensusArgs(ctypes.Structure):
    _fields_ = [("gx", _i32), ("gy", _i32)]


class MatvecArgs(ctypes.Structure):
    _fields_ = [("A", _vp), ("lda", _i64), ("m", _i32), ("n", _i32), ("x", _vp), ("y", _vp)]


class AtaxArgs(ctypes.Structure):
    _fields_ = [("A", _vp), ("lda", _i64), ("m", _i32), ("n", _i32), ("x", _vp), ("tmp", _vp), ("y", _vp)]


class BicgArgs(ctypes.Structure):
    _fields_ = [("A", _vp), ("lda", _i64), ("m", _i32), ("n", _i32), ("p", _vp), ("r", _vp), ("q", _vp), ("s", _vp)]


class MvtArgs(ctypes.Structure):
    _fields_ = [("A", _vp), ("lda", _i64), ("m", _i32), ("n", _i32), ("y1", _vp), ("y2", _vp), ("x1", _vp), ("x2", _vp)]


class Jacobi5Args(ctypes.Structure):
    _fields_ = [("a", _vp), ("b", _vp), ("ld", _i64), ("rows", _i32), ("cols", _i32), ("iters", _i32),
                ("result_is_b", _vp), ("row_lo", _i32), ("row_hi", _i32), ("fuse", _i32), ("tile_rows", _i32)]


class Jacobi5HaloArgs(ctypes.Structure):
    _fields_ = [("a", _vp), ("b", _vp), ("ld", _i64), ("rows", _i32), ("cols", _i32), ("iters", _i32),
                ("sweep0", _i32), ("result_is_b", _vp), ("ll", _vp), ("up_ll", _vp), ("dn_ll", _vp), ("status", _vp)]


class Conv2dArgs(ctypes.Structure):
    _fields_ = [("inp", _vp), ("out", _vp), ("ld", _i64), ("rows", _i32), ("cols", _i32), ("R", _i32), ("w", _vp)]


class SpmvArgs(ctypes.Structure):
    _fields_ = [("rows", _i32), ("cols", _i32), ("nnz", _i64), ("row_ptr", _vp), ("col", _vp), ("val", _vp),
                ("x", _vp), ("y", _vp), ("part", _vp), ("hot", _vp), ("xh", _vp), ("n_hot", _i32)]


_lib = None


def lib():
    """Load libctaclust.so (raises if it was not built: no fallback path)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise CtaclustError(-6, f"{LIB_PATH} not built (run `make` or __graft_entry__.build())")
        L = ctypes.CDLL(LIB_PATH)
        for name in EXPORTS:
            getattr(L, name)   # fail loudly on a missing export
        L.cc_status_string.restype = ctypes.c_char_p
        L.cc_last_error.restype = ctypes.c_char_p
        L.cc_version.restype = ctypes.c_char_p
        _lib = L
    return _lib


def _check(status: int):
    if status != 0:
        raise CtaclustError(status, lib().cc_last_error().decode())


def version() -> str:
    return lib().cc_version().decode()


# ---- device facts -----------------------------------------------------------
def device_info(device: int = 0) -> dict:
    n, span, l2 = _i32(), _i32(), _i32()
    _check(lib().cc_device_info(_i32(device), ctypes.byref(n), ctypes.byref(span), ctypes.byref(l2)))
    return {"num_sms": n.value, "smid_span": span.value, "l2_bytes": l2.value}


def sm_rank_table(device: int = 0) -> np.ndarray:
    span = _i32()
    _check(lib().cc_sm_rank_table(_i32(device), None, _i32(0), ctypes.byref(span)))
    out = np.zeros(span.value, dtype=np.int32)
    _check(lib().cc_sm_rank_table(_i32(device), out.ctypes.data_as(_vp), _i32(span.value), ctypes.byref(span)))
    return out


def max_agents(kernel, device: int = 0) -> int:
    k = KERNELS[kernel] if isinstance(kernel, str) else kernel
    out = _i32()
    _check(lib().cc_max_agents(_i32(k), _i32(device), ctypes.byref(out)))
    return out.value


# ---- planner ------------------------------------------------------------------
class Plan:
    """A cluster partition of a gx x gy logical grid (cc_plan)."""

    def __init__(self, gx: int, gy: int, order="row", num_clusters: int = 0, tile=(1, 1),
                 user_order=None, device: int | None = 0):
        o = ORDERS[order] if isinstance(order, str) else int(order)
        self._user = None
        if user_order is not None:
            self._user = np.ascontiguousarray(user_order, dtype=np.int32)
        d = PlanDesc(gx, gy, o, int(tile[0]), int(tile[1]), num_clusters,
                     self._user.ctypes.data if self._user is not None else None,
                     -1 if device is None else device)
        h = _vp()
        _check(lib().cc_plan_create(ctypes.byref(d), ctypes.byref(h)))
        self.handle = h
        self.gx, self.gy, self.order, self.device = gx, gy, o, device
        V, M, q, r = _i64(), _i32(), _i32(), _i32()
        _check(lib().cc_plan_info(h, ctypes.byref(V), ctypes.byref(M), ctypes.byref(q), ctypes.byref(r)))
        self.V, self.M, self.q, self.r = V.value, M.value, q.value, r.value

    def table(self):
        perm = np.zeros(self.V, dtype=np.int32)
        off = np.zeros(self.M + 1, dtype=np.int32)
        _check(lib().cc_plan_table(self.handle, perm.ctypes.data_as(_vp), off.ctypes.data_as(_vp)))
        return perm, off

    def lookup(self, v: int):
        w, i = _i32(), _i32()
        _check(lib().cc_plan_lookup(self.handle, _i32(v), ctypes.byref(w), ctypes.byref(i)))
        return w.value, i.value

    def invert(self, w: int, i: int) -> int:
        v = _i32()
        _check(lib().cc_plan_invert(self.handle, _i32(w), _i32(i), ctypes.byref(v)))
        return v.value

    def close(self):
        if getattr(self, "handle", None):
            lib().cc_plan_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


# ---- launch --------------------------------------------------------------------
def _ptr(t):
    return None if t is None else t.data_ptr()


def _stream(stream):
    import torch
    s = torch.cuda.current_stream() if stream is None else stream
    return s.cuda_stream


L2_HINTS = {"none": 0, "stream_first": 1, "reuse_last": 2, "both": 3, "halo_last": 4, "halo_last_stream_first": 5}


def make_opts(backend="agent", active_agents=0, max_agents=0, stages=0, batch=0, staging=0, steal=1,
              cluster_size=2, census=None, exec_sm=None, map=None, l2_hint=0, carveout=-1) -> LaunchOpts:
    b = BACKENDS[backend] if isinstance(backend, str) else int(backend)
    st = STAGINGS.get(staging, staging) if isinstance(staging, str) else int(staging)
    h = L2_HINTS[l2_hint] if isinstance(l2_hint, str) else int(l2_hint)
    return LaunchOpts(b, active_agents, max_agents, int(stages), int(batch), st, int(steal), cluster_size,
                      _ptr(census), _ptr(exec_sm), _ptr(map), h, int(carveout))


def kernel_grid(kernel, args) -> tuple[int, int]:
    k = KERNELS[kernel] if isinstance(kernel, str) else kernel
    gx, gy = _i32(), _i32()
    _check(lib().cc_kernel_grid(_i32(k), ctypes.byref(args), ctypes.byref(gx), ctypes.byref(gy)))
    return gx.value, gy.value


def launch(plan: Plan, kernel, args, opts: LaunchOpts | None = None, stream=None) -> int:
    """cc_launch; returns the number of kernels queued."""
    k = KERNELS[kernel] if isinstance(kernel, str) else kernel
    n = _i32()
    _check(lib().cc_launch(plan.handle, _i32(k), ctypes.byref(args),
                           ctypes.byref(opts) if opts is not None else None,
                           _vp(_stream(stream)), ctypes.byref(n)))
    return n.value


def _lda(A):
    assert A.dim() == 2 and A.stride(1) == 1, "row-major 2D tensor expected"
    return A.stride(0)


def matvec_args(A, x, y, m=None, n=None) -> MatvecArgs:
    m = A.shape[0] if m is None else m
    n = A.shape[1] if n is None else n
    return MatvecArgs(A.data_ptr(), _lda(A), m, n, x.data_ptr(), y.data_ptr())


def atax_args(A, x, tmp, y, m=None, n=None) -> AtaxArgs:
    m = A.shape[0] if m is None else m
    n = A.shape[1] if n is None else n
    return AtaxArgs(A.data_ptr(), _lda(A), m, n, x.data_ptr(), tmp.data_ptr(), y.data_ptr())


def bicg_args(A, p, r, q, s, m=None, n=None) -> BicgArgs:
    m = A.shape[0] if m is None else m
    n = A.shape[1] if n is None else n
    return BicgArgs(A.data_ptr(), _lda(A), m, n, p.data_ptr(), r.data_ptr(), q.data_ptr(), s.data_ptr())


def mvt_args(A, y1, y2, x1, x2, m=None, n=None) -> MvtArgs:
    m = A.shape[0] if m is None else m
    n = A.shape[1] if n is None else n
    return MvtArgs(A.data_ptr(), _lda(A), m, n, y1.data_ptr(), y2.data_ptr(), x1.data_ptr(), x2.data_ptr())


def jacobi5_args(a, b, iters, rows=None, cols=None, row_window=None, fuse=1,
                 tile_rows=0) -> tuple[Jacobi5Args, ctypes.c_int32]:
    """`row_window` = (row_lo, row_hi): write only output rows [row_lo, row_hi).
    `fuse`: sweeps per launch (1-4; 1-8 for jacobi5_wave); `tile_rows`:
    jacobi5_wave's logical CTA height (0 = 64)."""
    flag = _i32(0)
    rows = a.shape[0] if rows is None else rows
    cols = a.shape[1] if cols is None else cols
    lo, hi = (0, 0) if row_window is None else (int(row_window[0]), int(row_window[1]))
    if _lda(b) != _lda(a):
        raise CtaclustError(-1, f"jacobi5: a and b share one leading dimension (got {_lda(a)} and {_lda(b)})")
    args = Jacobi5Args(a.data_ptr(), b.data_ptr(), _lda(a), rows, cols, iters, ctypes.addressof(flag), lo, hi,
                       int(fuse), int(tile_rows))
    args._keep = flag            # result_is_b points into it: it must live as long as the struct
    return args, flag


def jacobi5_halo_args(a, b, iters, sweep0=0, ll=None, up_ll=None, dn_ll=None, status=None):
    """Args of one slab's fused-halo sweeps (CC_K_JACOBI5_HALO).  `ll`: this
    slab's LL buffer (int64 tensor of 4 * ldl words); `up_ll` / `dn_ll`: the
    neighbours' LL buffers as addresses valid in this process (same-device
    tensors' data_ptr(), or cc_ipc_open results), or None.  Returns (args,
    result_is_b flag)."""
    flag = _i32(0)
    args = Jacobi5HaloArgs(a.data_ptr(), b.data_ptr(), _lda(a), a.shape[0], a.shape[1], iters, sweep0,
                           ctypes.addressof(flag), _ptr(ll), up_ll, dn_ll, _ptr(status))
    args._keep = flag
    return args, flag


def ll_words(cols: int) -> int:
    """Words of a slab's LL buffer: 2 parities x 2 sides x cols rounded up to 32."""
    return 4 * ((cols + 31) & ~31)


def peer_access(device: int, peer: int):
    _check(lib().cc_peer_access(_i32(device), _i32(peer)))


def l2_persist(t, hit_ratio: float = 1.0, stream=None):
    """cc_l2_persist: keep device tensor t (or None: clear) L2-persisting for
    launches on `stream`."""
    ptr, nbytes = (None, 0) if t is None else (t.data_ptr(), t.numel() * t.element_size())
    _check(lib().cc_l2_persist(_vp(_stream(stream)), _vp(ptr), ctypes.c_size_t(nbytes), ctypes.c_float(hit_ratio)))


def ipc_handle(t) -> tuple[bytes, int]:
    """cc_ipc_handle: (64-byte handle of the allocation holding device tensor t,
    t's byte offset in that allocation)."""
    buf = ctypes.create_string_buffer(64)
    off = ctypes.c_uint64(0)
    _check(lib().cc_ipc_handle(_vp(t.data_ptr()), buf, ctypes.byref(off)))
    return buf.raw, off.value


def ipc_open(handle: bytes, device: int = 0) -> int:
    out = _vp()
    hb = ctypes.create_string_buffer(bytes(handle), 64)
    _check(lib().cc_ipc_open(hb, _i32(device), ctypes.byref(out)))
    return out.value


def ipc_close(ptr: int):
    _check(lib().cc_ipc_close(_vp(ptr)))


def conv2d_args(inp, out, w, rows=None, cols=None) -> tuple[Conv2dArgs, np.ndarray]:
    w = np.ascontiguousarray(np.asarray(w, dtype=np.float32))
    K = w.shape[0]
    rows = inp.shape[0] if rows is None else rows
    cols = inp.shape[1] if cols is None else cols
    if _lda(out) != _lda(inp):
        raise CtaclustError(-1, f"conv2d: in and out share one leading dimension (got {_lda(inp)} and {_lda(out)})")
    args = Conv2dArgs(inp.data_ptr(), out.data_ptr(), _lda(inp), rows, cols, K // 2, w.ctypes.data)
    args._keep = w               # the filter is read from this host array at launch
    return args, w


class Hist64Args(ctypes.Structure):
    _fields_ = [("data", _vp), ("n", _i64), ("counts", _vp)]


def hist64_args(data, counts) -> Hist64Args:
    return Hist64Args(_ptr(data), int(data.numel()), _ptr(counts))


def spmv_args(row_ptr, col, val, x, y, part=None) -> SpmvArgs:
    rows = row_ptr.numel() - 1
    return SpmvArgs(rows, x.numel(), col.numel(), row_ptr.data_ptr(), col.data_ptr(), val.data_ptr(),
                    x.data_ptr(), y.data_ptr(), _ptr(part))


def l1_reuse_probe(ctas: int, stagger_cycles: int, inp, smid, ticks, sink, stream=None):
    """cc_l1_reuse_probe: Listing 3 microbenchmark (device tensors, caller-owned)."""
    _check(lib().cc_l1_reuse_probe(_i32(ctas), _i32(stagger_cycles), _vp(inp.data_ptr()), _vp(smid.data_ptr()),
                                   _vp(ticks.data_ptr()), _vp(sink.data_ptr()), _vp(_stream(stream))))


def spmv_partition(args: SpmvArgs, part, stream=None):
    _check(lib().cc_spmv_partition(ctypes.byref(args), _vp(part.data_ptr()), _vp(_stream(stream))))


def spmv_inspect(args: SpmvArgs, max_hot: int, hot, col_hot, scratch, stream=None) -> int:
    """cc_spmv_inspect: hub columns of the plain CSR in `args` into `hot` and the
    encoded column array `col_hot` (device tensors); returns the slots used."""
    n = _i32()
    _check(lib().cc_spmv_inspect(ctypes.byref(args), _i32(max_hot), _vp(_ptr(hot)), _vp(_ptr(col_hot)),
                                 _vp(scratch.data_ptr()), ctypes.byref(n), _vp(_stream(stream))))
    return n.value


# ---- multi-GPU exchange steps (NCCL, one process per GPU) ---------------------
class Comm:
    """cc_comm: an NCCL communicator owned by the library.  Rank 0 creates the
    unique id (`Comm.unique_id()`), shares it out of band (torch.distributed
    broadcast), then every rank constructs `Comm(uid, nranks, rank, device)`."""

    @staticmethod
    def unique_id() -> bytes:
        buf = ctypes.create_string_buffer(128)
        _check(lib().cc_comm_unique_id(buf))
        return buf.raw

    def __init__(self, uid: bytes, nranks: int, rank: int, device: int = 0):
        h = _vp()
        idb = ctypes.create_string_buffer(bytes(uid), 128)
        _check(lib().cc_comm_init(idb, _i32(nranks), _i32(rank), _i32(device), ctypes.byref(h)))
        self.handle, self.nranks, self.rank = h, nranks, rank

    def halo_exchange(self, slab, halo: int, stream=None):
        """Refresh the halo rows of a local slab (rows x cols, row-major torch tensor)."""
        _check(lib().cc_halo_exchange(self.handle, _vp(slab.data_ptr()), _i64(slab.stride(0)), _i32(slab.shape[0]),
                                      _i32(slab.shape[1]), _i32(halo), _vp(_stream(stream))))

    def allreduce_sum(self, t, stream=None):
        _check(lib().cc_allreduce_sum(self.handle, _vp(t.data_ptr()), ctypes.c_size_t(t.numel()), _vp(_stream(stream))))

    def allgather(self, send, recv, stream=None):
        _check(lib().cc_allgather(self.handle, _vp(send.data_ptr()), _vp(recv.data_ptr()),
                                  ctypes.c_size_t(send.numel()), _vp(_stream(stream))))

    def close(self):
        if getattr(self, "handle", None):
            lib().cc_comm_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
