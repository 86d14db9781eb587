"""Thin ctypes binding of libhpccg.so (include/hpccg.h).

Argument marshalling only: every step of the path runs in the library's
sm_100a kernels.  There is no CPU fallback -- if ``libhpccg.so`` is missing or
fails to load, every entry point raises.  The module-level functions carry the
C names (``hpccg_generate``, ``hpccg_spmv``, ...); ``Context`` / ``Problem``
wrap them for convenience.  torch is used only for device memory and streams:
device-vector arguments may be CUDA float64 torch tensors (contiguous) or raw
device pointers (int).
"""
from __future__ import annotations

import ctypes
import os
import re
import threading

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("HPCCG_LIB") or os.path.join(_PKG, "libhpccg.so")  # override: A/B tools
HEADER = os.path.join(os.path.dirname(_PKG), "include", "hpccg.h")

HPCCG_OK = 0
HPCCG_EINVAL = -1
HPCCG_ENOMEM = -2
HPCCG_ECUDA = -3
HPCCG_ENCCL = -4
HPCCG_ENOTSUP = -5
HPCCG_UNIQUE_ID_BYTES = 128
HPCCG_VEC_X, HPCCG_VEC_B, HPCCG_VEC_XEXACT = 0, 1, 2
HPCCG_TRI_X, HPCCG_TRI_B, HPCCG_TRI_R, HPCCG_TRI_P = 0, 1, 2, 3
HPCCG_TRI_A0, HPCCG_TRI_A1, HPCCG_TRI_A2 = 4, 5, 6
HPCCG_OPT_GRAPH, HPCCG_OPT_POLL, HPCCG_OPT_TIMING = 0, 1, 2
HPCCG_OPT_SPMV_MINB, HPCCG_OPT_WHILE, HPCCG_OPT_L2_PERSIST, HPCCG_OPT_VEC_WAVES = 3, 4, 5, 6
HPCCG_OPT_SPMV_ROWS, HPCCG_OPT_VEC_UNROLL = 7, 8
HPCCG_OPT_PERSISTENT, HPCCG_OPT_PERSIST_ROWS, HPCCG_OPT_PDL = 9, 10, 11
HPCCG_OPT_CLUSTER_ROWS, HPCCG_OPT_SMEM_SOLVE, HPCCG_OPT_TRACE = 12, 13, 14
HPCCG_OPT_WHILE_UNROLL, HPCCG_OPT_CG_VARIANT, HPCCG_OPT_FINISHER_FREE = 15, 16, 17
HPCCG_OPT_SMEM_THREADS, HPCCG_OPT_HALO_PEER, HPCCG_OPT_SERPENTINE = 18, 19, 20
HPCCG_OPT_SPMV_FORMAT, HPCCG_OPT_PEER_TIMEOUT_MS, HPCCG_OPT_DEFER_X = 21, 22, 23
HPCCG_OPT_FUSE_PSPMV, HPCCG_OPT_PS_LEAD, HPCCG_OPT_SPMV_TRIPS = 24, 25, 26
HPCCG_OPT_PAP_CLUSTER, HPCCG_OPT_SPMV_SLICED, HPCCG_OPT_SPMV_CLUSTER = 27, 28, 29
HPCCG_OPT_SMEM_HALO = 30

_lock = threading.Lock()
_lib = None


class HpccgError(RuntimeError):
    def __init__(self, code: int, where: str, detail: str):
        super().__init__(f"{where}: {detail or ''} [{code}]")
        self.code = code


class hpccg_stats(ctypes.Structure):
    _fields_ = [("total_ms", ctypes.c_double), ("spmv_ms", ctypes.c_double),
                ("update_ms", ctypes.c_double), ("pupdate_ms", ctypes.c_double),
                ("allreduce_ms", ctypes.c_double), ("exchange_ms", ctypes.c_double),
                ("spmv_launches", ctypes.c_int64), ("iterations", ctypes.c_int64),
                ("kernel_launches", ctypes.c_int64), ("l2_persist_bytes", ctypes.c_int64),
                ("graph_mode", ctypes.c_int64), ("x_deferred", ctypes.c_int64),
                ("ps_fused", ctypes.c_int64)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


_vp, _i, _i64, _d = ctypes.c_void_p, ctypes.c_int, ctypes.c_int64, ctypes.c_double
_pi64 = ctypes.POINTER(ctypes.c_int64)
_SIGS = {
    "hpccg_strerror": ([_i], ctypes.c_char_p),
    "hpccg_last_error": ([], ctypes.c_char_p),
    "hpccg_version": ([], ctypes.c_char_p),
    "hpccg_launch_count": ([_vp, _pi64], _i),
    "hpccg_unique_id": ([_vp], _i),
    "hpccg_init": ([ctypes.POINTER(_vp), _i, _vp, _i, _i, _vp], _i),
    "hpccg_init_loopback": ([ctypes.POINTER(_vp), _i, _vp, _i], _i),
    "hpccg_init_peer": ([ctypes.POINTER(_vp), _i, _vp, _i, _i], _i),
    "hpccg_peer_export": ([_vp, _vp], _i),
    "hpccg_peer_attach": ([_vp, _vp], _i),
    "hpccg_ctx_info": ([_vp, ctypes.POINTER(_i), ctypes.POINTER(_i), ctypes.POINTER(_i)], _i),
    "hpccg_finalize": ([_vp], None),
    "hpccg_generate": ([_vp, _i, _i, _i, ctypes.POINTER(_vp)], _i),
    "hpccg_info": ([_vp, _pi64, _pi64, _pi64, _pi64, _pi64], _i),
    "hpccg_vec": ([_vp, _i, ctypes.POINTER(_vp)], _i),
    "hpccg_set_vec": ([_vp, _i, _vp], _i),
    "hpccg_get_vec": ([_vp, _i, _vp], _i),
    "hpccg_copy_matrix": ([_vp, _i, _vp, _vp], _i),
    "hpccg_set_option": ([_vp, _i, _i64], _i),
    "hpccg_spmv": ([_vp, _vp, _vp], _i),
    "hpccg_ddot": ([_vp, _i64, _vp, _vp, ctypes.POINTER(_d)], _i),
    "hpccg_waxpby": ([_vp, _i64, _d, _vp, _d, _vp, _vp], _i),
    "hpccg_solve": ([_vp, _i, _d, ctypes.POINTER(_i), ctypes.POINTER(_d), _vp], _i),
    "hpccg_get_stats": ([_vp, ctypes.POINTER(hpccg_stats)], _i),
    "hpccg_get_trace": ([_vp, _vp, _i64], _i),
    "hpccg_maxabsdiff": ([_vp, ctypes.POINTER(_d)], _i),
    "hpccg_free": ([_vp], None),
    "hpccg_waxpby2d": ([_vp, _i64, _i64, _i64, _d, _vp, _d, _vp, _vp], _i),
    "hpccg_ddot2d": ([_vp, _i64, _i64, _i64, _vp, _vp, ctypes.POINTER(_d)], _i),
    "hpccg_lbm_create": ([_vp, _i, ctypes.POINTER(_vp)], _i),
    "hpccg_lbm_set": ([_vp, _i, _vp], _i),
    "hpccg_lbm_get": ([_vp, _i, _vp], _i),
    "hpccg_lbm_run": ([_vp, _i, _d, _i, ctypes.POINTER(_d)], _i),
    "hpccg_lbm_free": ([_vp], None),
    "hpccg_tri_generate": ([_vp, _i64, ctypes.POINTER(_vp)], _i),
    "hpccg_tri_vec": ([_vp, _i, ctypes.POINTER(_vp)], _i),
    "hpccg_tri_spmv": ([_vp, _vp, _vp], _i),
    "hpccg_tri_solve": ([_vp, _i, _d, _i, ctypes.POINTER(_i), ctypes.POINTER(_d),
                         ctypes.POINTER(_d)], _i),
    "hpccg_tri_free": ([_vp], None),
}


def header_symbols(path: str = HEADER):
    """Every function the C header declares (HPCCG_API ... name(...))."""
    txt = open(path).read()
    return sorted(set(re.findall(r"HPCCG_API[^;(]*?\b(hpccg_\w+)\s*\(", txt)))


def lib():
    """Load libhpccg.so (raises if it is missing: there is no fallback)."""
    global _lib
    with _lock:
        if _lib is not None:
            return _lib
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} is missing: build it with "
                               "`python -c 'import __graft_entry__ as g; g.build()'`")
        L = ctypes.CDLL(LIB_PATH)
        for name, (args, res) in _SIGS.items():
            f = getattr(L, name)
            f.argtypes = args
            f.restype = res
        _lib = L
        return L


def _check(rc: int, where: str):
    if rc != HPCCG_OK:
        L = lib()
        raise HpccgError(rc, where, (L.hpccg_last_error() or b"").decode())


def _ptr(t) -> int:
    """Device pointer of a CUDA tensor (contiguous float64) or a raw int."""
    if isinstance(t, int):
        return t
    import torch
    if not isinstance(t, torch.Tensor):
        raise TypeError("expected a torch CUDA tensor or a raw device pointer")
    if not t.is_cuda or t.dtype != torch.float64 or not t.is_contiguous():
        raise TypeError("device vectors must be contiguous CUDA float64 tensors")
    return t.data_ptr()


def _torch_sync():
    """Order the library's stream after torch's pending work on user tensors."""
    try:
        import torch
        if torch.cuda.is_available() and torch.cuda.is_initialized():
            torch.cuda.current_stream().synchronize()
    except Exception:  # pragma: no cover
        pass


class _CudaArray:
    def __init__(self, ptr: int, n: int):
        self.__cuda_array_interface__ = {"shape": (n,), "typestr": "<f8", "data": (ptr, False),
                                         "version": 3, "strides": None}


def device_view(ptr: int, n: int):
    """torch view (no copy) of n doubles of library-owned device memory."""
    import torch
    return torch.as_tensor(_CudaArray(ptr, n), device="cuda")


# ------------------------------------------------------------ C-named calls

def hpccg_version() -> str:
    return lib().hpccg_version().decode()


def hpccg_strerror(code: int) -> str:
    return lib().hpccg_strerror(code).decode()


def hpccg_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(HPCCG_UNIQUE_ID_BYTES)
    _check(lib().hpccg_unique_id(buf), "hpccg_unique_id")
    return buf.raw


def hpccg_init(device: int = 0, stream: int | None = None, rank: int = 0, nranks: int = 1,
               unique_id: bytes | None = None) -> int:
    h = _vp()
    uid = None
    if unique_id is not None:
        uid = ctypes.create_string_buffer(bytes(unique_id), HPCCG_UNIQUE_ID_BYTES)
    _check(lib().hpccg_init(ctypes.byref(h), device, stream or None, rank, nranks, uid),
           "hpccg_init")
    return h.value


def hpccg_init_loopback(device: int = 0, stream: int | None = None, nranks: int = 2) -> int:
    h = _vp()
    _check(lib().hpccg_init_loopback(ctypes.byref(h), device, stream or None, nranks),
           "hpccg_init_loopback")
    return h.value


def hpccg_init_peer(device: int = 0, stream: int | None = None, rank: int = 0,
                    nranks: int = 2) -> int:
    h = _vp()
    _check(lib().hpccg_init_peer(ctypes.byref(h), device, stream or None, rank, nranks),
           "hpccg_init_peer")
    return h.value


HPCCG_PEER_BLOB_BYTES = 256


def hpccg_peer_export(prob: int) -> bytes:
    buf = ctypes.create_string_buffer(HPCCG_PEER_BLOB_BYTES)
    _check(lib().hpccg_peer_export(prob, buf), "hpccg_peer_export")
    return buf.raw


def hpccg_peer_attach(prob: int, blobs) -> None:
    data = b"".join(bytes(b) for b in blobs)
    if any(len(b) != HPCCG_PEER_BLOB_BYTES for b in blobs):
        raise ValueError("peer blobs must be %d bytes each" % HPCCG_PEER_BLOB_BYTES)
    buf = ctypes.create_string_buffer(data, len(data))
    _check(lib().hpccg_peer_attach(prob, buf), "hpccg_peer_attach")


def hpccg_finalize(ctx: int) -> None:
    lib().hpccg_finalize(ctx)


def hpccg_generate(ctx: int, nx: int, ny: int, nz: int) -> int:
    h = _vp()
    _check(lib().hpccg_generate(ctx, nx, ny, nz, ctypes.byref(h)), "hpccg_generate")
    return h.value


def hpccg_info(prob: int) -> dict:
    v = [ctypes.c_int64() for _ in range(5)]
    _check(lib().hpccg_info(prob, *[ctypes.byref(x) for x in v]), "hpccg_info")
    keys = ("nrow_local", "ncol_local", "nnz_local", "nrow_global", "nnz_global")
    return {k: x.value for k, x in zip(keys, v)}


def _sync_if_tensors(*args):
    """Order after torch's pending work only when torch tensors are passed
    (raw device pointers: the caller owns the ordering)."""
    if any(not isinstance(a, int) for a in args):
        _torch_sync()


def hpccg_spmv(prob: int, x, y) -> None:
    _sync_if_tensors(x, y)
    _check(lib().hpccg_spmv(prob, _ptr(x), _ptr(y)), "hpccg_spmv")


def hpccg_ddot(ctx: int, n: int, x, y) -> float:
    _sync_if_tensors(x, y)
    r = ctypes.c_double()
    _check(lib().hpccg_ddot(ctx, n, _ptr(x), _ptr(y), ctypes.byref(r)), "hpccg_ddot")
    return r.value


def hpccg_waxpby(ctx: int, n: int, alpha: float, x, beta: float, y, w) -> None:
    _sync_if_tensors(x, y, w)
    _check(lib().hpccg_waxpby(ctx, n, float(alpha), _ptr(x), float(beta), _ptr(y), _ptr(w)),
           "hpccg_waxpby")


def hpccg_waxpby2d(ctx: int, m: int, n: int, ld: int, alpha: float, x, beta: float, y, w) -> None:
    _sync_if_tensors(x, y, w)
    _check(lib().hpccg_waxpby2d(ctx, m, n, ld, float(alpha), _ptr(x), float(beta), _ptr(y),
                                _ptr(w)), "hpccg_waxpby2d")


def hpccg_ddot2d(ctx: int, m: int, n: int, ld: int, x, y) -> float:
    _sync_if_tensors(x, y)
    r = ctypes.c_double()
    _check(lib().hpccg_ddot2d(ctx, m, n, ld, _ptr(x), _ptr(y), ctypes.byref(r)), "hpccg_ddot2d")
    return r.value


def hpccg_solve(prob: int, max_iter: int, tol: float) -> dict:
    ni, nr = ctypes.c_int(), ctypes.c_double()
    times = (ctypes.c_double * 6)()
    _check(lib().hpccg_solve(prob, max_iter, float(tol), ctypes.byref(ni), ctypes.byref(nr),
                             times), "hpccg_solve")
    return {"niters": ni.value, "normr": nr.value, "times": list(times)}


def hpccg_get_stats(prob: int) -> dict:
    s = hpccg_stats()
    _check(lib().hpccg_get_stats(prob, ctypes.byref(s)), "hpccg_get_stats")
    return s.as_dict()


def hpccg_maxabsdiff(prob: int) -> float:
    r = ctypes.c_double()
    _check(lib().hpccg_maxabsdiff(prob, ctypes.byref(r)), "hpccg_maxabsdiff")
    return r.value


def hpccg_free(prob: int) -> None:
    lib().hpccg_free(prob)


# --------------------------------------------------------------- wrappers

class Context:
    """A device + stream + communicator (single GPU, NCCL rank, or loopback)."""

    def __init__(self, device: int = 0, stream: int | None = None, rank: int = 0,
                 nranks: int = 1, unique_id: bytes | None = None, loopback: bool = False,
                 peer: bool = False):
        if loopback:
            self.handle = hpccg_init_loopback(device, stream, nranks)
        elif peer:      # peer-only (no NCCL): attach problems with peer_export / peer_attach
            self.handle = hpccg_init_peer(device, stream, rank, nranks)
        else:
            self.handle = hpccg_init(device, stream, rank, nranks, unique_id)
        self.kind = "loopback" if loopback else "peer" if peer else "nccl" if nranks > 1 or unique_id \
            else "single"
        i = self.info()
        self.rank, self.nranks, self.nslabs = i["rank"], i["nranks"], i["nslabs"]

    def info(self) -> dict:
        """hpccg_ctx_info (NCCL contexts: the communicator's own rank / count)."""
        r, n, s = ctypes.c_int(), ctypes.c_int(), ctypes.c_int()
        _check(lib().hpccg_ctx_info(self.handle, ctypes.byref(r), ctypes.byref(n),
                                    ctypes.byref(s)), "hpccg_ctx_info")
        return {"rank": r.value, "nranks": n.value, "nslabs": s.value, "kind": self.kind}

    def ddot(self, n: int, x, y) -> float:
        return hpccg_ddot(self.handle, n, x, y)

    def waxpby(self, n: int, alpha: float, x, beta: float, y, w) -> None:
        hpccg_waxpby(self.handle, n, alpha, x, beta, y, w)

    def waxpby2d(self, m: int, n: int, ld: int, alpha: float, x, beta: float, y, w) -> None:
        hpccg_waxpby2d(self.handle, m, n, ld, alpha, x, beta, y, w)

    def ddot2d(self, m: int, n: int, ld: int, x, y) -> float:
        return hpccg_ddot2d(self.handle, m, n, ld, x, y)

    @property
    def launch_count(self) -> int:
        c = ctypes.c_int64()
        _check(lib().hpccg_launch_count(self.handle, ctypes.byref(c)), "hpccg_launch_count")
        return c.value

    def close(self):
        if self.handle:
            hpccg_finalize(self.handle)
            self.handle = 0

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()


class Problem:
    """One rank's (or, loopback, all ranks') slab of the HPCCG problem."""

    def __init__(self, ctx: Context, nx: int, ny: int, nz: int):
        self.ctx = ctx
        self.nx, self.ny, self.nz = nx, ny, nz
        self.handle = hpccg_generate(ctx.handle, nx, ny, nz)
        self.info = hpccg_info(self.handle)

    @property
    def n(self) -> int:
        return self.info["nrow_local"]

    @property
    def ncol(self) -> int:
        return self.info["ncol_local"]

    def set_option(self, key: int, value: int) -> None:
        _check(lib().hpccg_set_option(self.handle, key, int(value)), "hpccg_set_option")

    def spmv(self, x, y) -> None:
        hpccg_spmv(self.handle, x, y)

    def solve(self, max_iter: int, tol: float) -> dict:
        return hpccg_solve(self.handle, max_iter, tol)

    def stats(self) -> dict:
        return hpccg_get_stats(self.handle)

    def maxabsdiff(self) -> float:
        return hpccg_maxabsdiff(self.handle)

    def peer_export(self) -> bytes:
        """This rank's CUDA-IPC blob (one slab per process)."""
        return hpccg_peer_export(self.handle)

    def peer_attach(self, blobs) -> None:
        """Map every rank's blob (rank order) and switch HALO_PEER on."""
        hpccg_peer_attach(self.handle, blobs)

    def trace(self, k: int) -> np.ndarray:
        """[k, 3, 2] uint64 ns: (start, end) of p update / SpMV / update per iteration."""
        out = np.zeros(6 * k, dtype=np.uint64)
        _check(lib().hpccg_get_trace(self.handle, out.ctypes.data, k), "hpccg_get_trace")
        return out.reshape(k, 3, 2)

    def get_vec(self, which: int, out: np.ndarray | None = None) -> np.ndarray:
        """Host copy (nslabs * n doubles).  `out` may be a pinned buffer."""
        if out is None:
            out = np.empty(self.ctx.nslabs * self.n, dtype=np.float64)
        assert out.dtype == np.float64 and out.flags.c_contiguous
        assert out.size >= self.ctx.nslabs * self.n
        _check(lib().hpccg_get_vec(self.handle, which, out.ctypes.data), "hpccg_get_vec")
        return out

    def set_vec(self, which: int, src: np.ndarray) -> None:
        src = np.ascontiguousarray(src, dtype=np.float64)
        assert src.size >= self.ctx.nslabs * self.n
        _check(lib().hpccg_set_vec(self.handle, which, src.ctypes.data), "hpccg_set_vec")

    def get_vec_ptr(self, which: int, host_ptr: int) -> None:
        _check(lib().hpccg_get_vec(self.handle, which, host_ptr), "hpccg_get_vec")

    def set_vec_ptr(self, which: int, host_ptr: int) -> None:
        _check(lib().hpccg_set_vec(self.handle, which, host_ptr), "hpccg_set_vec")

    def vec_ptr(self, which: int) -> int:
        h = _vp()
        _check(lib().hpccg_vec(self.handle, which, ctypes.byref(h)), "hpccg_vec")
        return h.value

    def copy_matrix(self, slab: int = 0):
        """(val, col) host arrays, slot-major [27, n]."""
        n = self.n
        val = np.empty(27 * n, dtype=np.float64)
        col = np.empty(27 * n, dtype=np.int32)
        _check(lib().hpccg_copy_matrix(self.handle, slab, val.ctypes.data, col.ctypes.data),
               "hpccg_copy_matrix")
        return val.reshape(27, n), col.reshape(27, n)

    def free(self):
        if self.handle:
            hpccg_free(self.handle)
            self.handle = 0

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.free()


# ------------------------------------------------- f1: Fig. 12 tridiagonal CG

class Tri:
    """The paper's own CG workload (Fig. 12) on the device (hpccg_tri_*)."""

    def __init__(self, ctx: Context, n: int):
        self.ctx, self.n = ctx, n
        h = _vp()
        _check(lib().hpccg_tri_generate(ctx.handle, n, ctypes.byref(h)), "hpccg_tri_generate")
        self.handle = h.value

    def vec_ptr(self, which: int) -> int:
        h = _vp()
        _check(lib().hpccg_tri_vec(self.handle, which, ctypes.byref(h)), "hpccg_tri_vec")
        return h.value

    def spmv(self, x, y) -> None:
        _sync_if_tensors(x, y)
        _check(lib().hpccg_tri_spmv(self.handle, _ptr(x), _ptr(y)), "hpccg_tri_spmv")

    def solve(self, max_iter: int, tol: float, variant: int = 1) -> dict:
        it, cond, ms = ctypes.c_int(), ctypes.c_double(), ctypes.c_double()
        _check(lib().hpccg_tri_solve(self.handle, max_iter, float(tol), variant, ctypes.byref(it),
                                     ctypes.byref(cond), ctypes.byref(ms)), "hpccg_tri_solve")
        return {"iters": it.value, "cond": cond.value, "ms": ms.value}

    def view(self, which: int):
        """Zero-copy torch view of a device vector (valid until free())."""
        return device_view(self.vec_ptr(which), self.n)

    def get(self, which: int) -> np.ndarray:
        return self.view(which).cpu().numpy()

    def free(self):
        if self.handle:
            lib().hpccg_tri_free(self.handle)
            self.handle = 0

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.free()


# ------------------------------------------------------ f4: D2Q9 pull LBM

class Lbm:
    """The paper's D2Q9 pull LBM (Fig. 10) on the device (hpccg_lbm_*)."""

    def __init__(self, ctx: Context, size: int):
        self.ctx, self.S = ctx, size
        h = _vp()
        _check(lib().hpccg_lbm_create(ctx.handle, size, ctypes.byref(h)), "hpccg_lbm_create")
        self.handle = h.value

    def set(self, which: int, host: np.ndarray) -> None:
        host = np.ascontiguousarray(host, dtype=np.float64)
        assert host.size == 9 * self.S * self.S
        _check(lib().hpccg_lbm_set(self.handle, which, host.ctypes.data), "hpccg_lbm_set")

    def get(self, which: int) -> np.ndarray:
        out = np.empty(9 * self.S * self.S, dtype=np.float64)
        _check(lib().hpccg_lbm_get(self.handle, which, out.ctypes.data), "hpccg_lbm_get")
        return out

    def run(self, steps: int, tau: float, write_f: bool = False) -> float:
        ms = ctypes.c_double()
        _check(lib().hpccg_lbm_run(self.handle, steps, float(tau), int(write_f), ctypes.byref(ms)),
               "hpccg_lbm_run")
        return ms.value

    def free(self):
        if self.handle:
            lib().hpccg_lbm_free(self.handle)
            self.handle = 0

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.free()
