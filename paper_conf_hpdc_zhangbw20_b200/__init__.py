"""B200-native recursive Gram-Schmidt QR (RGSQR) -- Python binding of librgsqr.so.

Argument marshalling only: every step of the computation runs in the CUDA kernels of
``csrc/`` behind the C-ABI declared in ``include/rgsqr.h``.  There is no CPU or
PyTorch fallback: if the shared library is missing or no sm_100 GPU is present the
calls raise.

Matrices are column-major fp32, i.e. torch tensors of shape (rows, cols) with
``stride(0) == 1`` (``X.t().contiguous().t()`` or :func:`colmajor`), or numpy
``order='F'`` arrays for the host-pointer path (the library stages them).

Paper: Zhang, Baharlouei, Wu, HPDC'20 -- Algorithm 1, eq 8 panel
(P:L221-237), Algorithm 3 CGLS, section 3.3 reorthogonalisation,
section 3.4 low rank, section 3.5 scaling.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "librgsqr.so")

RG_OK, RG_BREAKDOWN, RG_NOT_CONVERGED, RG_NONFINITE, RG_CUDA_ERROR, RG_NCCL_ERROR, RG_NO_DEVICE, RG_ALLOC = range(8)

EXPORTS = [
    "rg_opts_default", "rg_create", "rg_set_stream", "rg_destroy", "rg_status_string", "rg_last_info",
    "rg_version", "rg_last_launches", "rg_nccl_load", "rg_comm_unique_id", "rg_comm_init", "rgsqr_factor", "orthogonalize",
    "ls_solve_refined", "lowrank_approx", "rg_profile_enable", "rg_profile_reset", "rg_profile_get",
    "rg_set_comm", "rg_vgroup_create", "rg_vgroup_destroy", "rg_set_vcomm", "rg_debug_gaussian", "rg_debug_philox", "lowrank_qrsvd",
]
RG_MAX_RANKS = 8

PROFILE_CLASSES = {"update": 0, "proj": 1, "panel": 2, "scale": 3, "cgls": 4, "other": 5}


class RGError(RuntimeError):
    def __init__(self, func, status, info=-1):
        self.status = status
        self.info = info
        msg = f"{func} failed: status {status}"
        try:
            msg += f" ({_lib().rg_status_string(status).decode()})"
        except Exception:
            pass
        if info >= 0:
            msg += f", column {info}"
        super().__init__(msg)


class rg_opts(ctypes.Structure):
    _fields_ = [("precision", ctypes.c_int), ("nb", ctypes.c_int), ("scale", ctypes.c_int),
                ("reortho", ctypes.c_int), ("split", ctypes.c_int), ("sync", ctypes.c_int),
                ("panel", ctypes.c_int), ("solver", ctypes.c_int)]


_LIB = None


def _lib():
    global _LIB
    if _LIB is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} is missing: run `python -c 'import __graft_entry__ as g; g.build()'` "
                              "(there is no fallback implementation)")
        L = ctypes.CDLL(LIB_PATH)
        vp, i64, i32, f64p = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int, ctypes.POINTER(ctypes.c_double)
        L.rg_opts_default.argtypes = [ctypes.POINTER(rg_opts)]
        L.rg_create.argtypes = [ctypes.POINTER(vp), i32, vp]
        L.rg_set_stream.argtypes = [vp, vp]
        L.rg_destroy.argtypes = [vp]
        L.rg_status_string.argtypes = [i32]
        L.rg_status_string.restype = ctypes.c_char_p
        L.rg_last_info.argtypes = [vp]
        L.rg_last_info.restype = i64
        L.rg_version.restype = ctypes.c_char_p
        L.rg_last_launches.argtypes = [vp]
        L.rg_last_launches.restype = i64
        L.rg_nccl_load.argtypes = [ctypes.c_char_p]
        L.rg_comm_unique_id.argtypes = [vp]
        L.rg_comm_init.argtypes = [vp, vp, i32, i32]
        L.rg_set_comm.argtypes = [vp, vp, i32, i32]
        L.rg_vgroup_create.argtypes = [ctypes.POINTER(vp), i32]
        L.rg_vgroup_destroy.argtypes = [vp]
        L.rg_set_vcomm.argtypes = [vp, vp, i32]
        L.rg_debug_gaussian.argtypes = [vp, i64, ctypes.c_uint64, vp]
        L.rg_debug_philox.argtypes = [vp, i64, ctypes.c_uint64, vp]
        L.rgsqr_factor.argtypes = [vp, i64, i64, vp, i64, vp, i64, vp, i64, ctypes.POINTER(rg_opts)]
        L.orthogonalize.argtypes = [vp, i64, i64, vp, i64, vp, i64, ctypes.c_double, i32,
                                    ctypes.POINTER(i32), f64p, ctypes.POINTER(rg_opts)]
        L.ls_solve_refined.argtypes = [vp, i64, i64, vp, i64, vp, vp, ctypes.c_double, i32,
                                       ctypes.POINTER(i32), f64p, ctypes.POINTER(rg_opts)]
        L.lowrank_approx.argtypes = [vp, i64, i64, vp, i64, i32, i32, i32, ctypes.c_uint64, vp, i64, vp, vp, i64,
                                     ctypes.POINTER(rg_opts)]
        L.lowrank_qrsvd.argtypes = [vp, i64, i64, vp, i64, i32, vp, i64, vp, vp, i64, ctypes.POINTER(rg_opts)]
        L.rg_profile_enable.argtypes = [vp, i32]
        L.rg_profile_reset.argtypes = [vp]
        L.rg_profile_get.argtypes = [vp, i32, f64p, ctypes.POINTER(i64), f64p, f64p]
        for name in EXPORTS:
            if getattr(L, name).restype is None and name not in ("rg_opts_default",):
                getattr(L, name).restype = i32
        L.rg_opts_default.restype = None
        _LIB = L
    return _LIB


def lib():
    return _lib()


def version() -> str:
    return _lib().rg_version().decode()


def make_opts(precision="fp16", nb=32, scale=True, reortho=-1, split=False, sync=True, panel="auto",
              solver="cgls") -> rg_opts:
    o = rg_opts()
    _lib().rg_opts_default(ctypes.byref(o))
    o.precision = {"fp16": 0, "bf16": 1}[precision] if isinstance(precision, str) else int(precision)
    o.nb = int(nb)
    o.scale = int(bool(scale))
    o.reortho = int(reortho)
    o.split = int(bool(split))
    o.sync = int(bool(sync))
    o.panel = {"auto": 0, "cholqr2": 0, "mgs": 1, "tsqr": 1}[panel] if isinstance(panel, str) else int(panel)
    o.solver = {"cgls": 0, "lsqr": 1}[solver] if isinstance(solver, str) else int(solver)
    return o


def colmajor(t):
    """Column-major copy of a 2-D torch tensor / numpy array (fp32)."""
    if isinstance(t, np.ndarray):
        return np.asfortranarray(t, dtype=np.float32)
    import torch
    return t.to(torch.float32).t().contiguous().t()


@dataclass
class _Mat:
    ptr: int
    rows: int
    cols: int
    ld: int
    host: bool


def _mat(x, name, dtype="float32") -> _Mat:
    if isinstance(x, np.ndarray):
        if x.dtype != np.dtype(dtype):
            raise TypeError(f"{name} must be {dtype}")
        if x.ndim == 1:
            return _Mat(x.ctypes.data, x.shape[0], 1, max(1, x.shape[0]), True)
        if x.strides[0] != x.itemsize:
            raise ValueError(f"{name} must be column-major (order='F')")
        ld = x.strides[1] // x.itemsize if x.shape[1] > 1 else x.shape[0]
        return _Mat(x.ctypes.data, x.shape[0], x.shape[1], max(ld, 1), True)
    import torch
    if not isinstance(x, torch.Tensor):
        raise TypeError(f"{name} must be a torch tensor or numpy array")
    want = {"float32": torch.float32, "float64": torch.float64}[dtype]
    if x.dtype != want:
        raise TypeError(f"{name} must be {want}")
    host = not x.is_cuda
    if x.dim() == 1:
        if x.stride(0) != 1:
            raise ValueError(f"{name} must be contiguous")
        return _Mat(x.data_ptr(), x.shape[0], 1, max(1, x.shape[0]), host)
    if x.stride(0) != 1 and x.shape[0] > 1:
        raise ValueError(f"{name} must be column-major (stride(0) == 1)")
    ld = x.stride(1) if x.shape[1] > 1 else x.shape[0]
    return _Mat(x.data_ptr(), x.shape[0], x.shape[1], max(ld, x.shape[0], 1), host)


class Handle:
    """Owns an rg_handle bound to a CUDA device and stream (default: torch's current stream)."""

    def __init__(self, device: int = 0, stream=None):
        self._h = ctypes.c_void_p()
        if stream is None:
            import torch
            stream = torch.cuda.current_stream(device).cuda_stream
        st = _lib().rg_create(ctypes.byref(self._h), int(device), ctypes.c_void_p(int(stream)))
        if st != RG_OK:
            raise RGError("rg_create", st)
        self.device = device
        self.rank, self.nranks = 0, 1

    @property
    def ptr(self):
        return self._h

    def close(self):
        if self._h:
            _lib().rg_destroy(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def set_stream(self, stream):
        _check("rg_set_stream", _lib().rg_set_stream(self._h, ctypes.c_void_p(int(stream))), self)

    def last_info(self) -> int:
        return int(_lib().rg_last_info(self._h))

    def last_launches(self) -> int:
        return int(_lib().rg_last_launches(self._h))

    # ---- multi-GPU (row-sharded) -------------------------------------------------------
    def init_comm(self, rank: int, nranks: int, group=None, nccl_path=None):
        """Create the library's NCCL communicator; the unique id is broadcast with
        torch.distributed (any backend) from rank 0."""
        import torch
        import torch.distributed as dist
        path = nccl_path or _find_nccl()
        st = _lib().rg_nccl_load(path.encode() if path else None)
        if st != RG_OK:
            raise RGError("rg_nccl_load", st)
        buf = (ctypes.c_char * 128)()
        if rank == 0:
            _check("rg_comm_unique_id", _lib().rg_comm_unique_id(buf), self)
        if nranks > 1:
            t = torch.tensor(list(bytearray(buf.raw)), dtype=torch.uint8)
            if dist.get_backend(group) == "nccl":
                t = t.cuda(self.device)
            dist.broadcast(t, src=0, group=group)
            ctypes.memmove(buf, bytes(t.cpu().tolist()), 128)
        _check("rg_comm_init", _lib().rg_comm_init(self._h, buf, int(rank), int(nranks)), self)
        self.rank, self.nranks = rank, nranks

    def set_comm(self, nccl_comm_ptr: int, rank: int, nranks: int):
        """Row-sharded mode on a caller-owned ncclComm_t (0 detaches)."""
        _check("rg_set_comm", _lib().rg_set_comm(self._h, ctypes.c_void_p(int(nccl_comm_ptr)), int(rank),
                                                 int(nranks)), self)
        self.rank, self.nranks = (rank, nranks) if nccl_comm_ptr else (0, 1)

    def attach_torch_comm(self, group=None):
        """Row-sharded mode on torch.distributed's own NCCL communicator (ProcessGroupNCCL of
        `group`, default the world) through rg_set_comm: no second communicator.  torch loads
        libnccl dynamically from nvidia/nccl/lib; the library dlopens the same file, so the
        ncclComm_t is valid for its calls.  Collectives of torch and of the library on this
        communicator must not overlap in time (synchronise between them)."""
        import torch
        import torch.distributed as dist
        pg = group or dist.distributed_c10d._get_default_group()
        backend = pg._get_backend(torch.device("cuda", self.device))
        dist.barrier(group=pg)          # the communicator exists once a collective has run
        torch.cuda.synchronize(self.device)
        path = _find_nccl()
        st = _lib().rg_nccl_load(path.encode() if path else None)
        if st != RG_OK:
            raise RGError("rg_nccl_load", st)
        self.set_comm(backend._comm_ptr(), dist.get_rank(pg), dist.get_world_size(pg))

    def set_vcomm(self, group, rank: int):
        """Attach to an in-process virtual-rank group (VGroup); None detaches."""
        _check("rg_set_vcomm", _lib().rg_set_vcomm(self._h, group.ptr if group is not None else None, int(rank)),
               self)
        self.rank, self.nranks = (rank, group.nranks) if group is not None else (0, 1)

    # ---- profiling -------------------------------------------------------------------------
    def profile(self, enable=True):
        _lib().rg_profile_enable(self._h, int(bool(enable)))

    def profile_reset(self):
        _lib().rg_profile_reset(self._h)

    def profile_get(self, cls):
        ms, fl, by = ctypes.c_double(), ctypes.c_double(), ctypes.c_double()
        n = ctypes.c_int64()
        c = PROFILE_CLASSES[cls] if isinstance(cls, str) else int(cls)
        _lib().rg_profile_get(self._h, c, ctypes.byref(ms), ctypes.byref(n), ctypes.byref(fl), ctypes.byref(by))
        return {"ms": ms.value, "launches": n.value, "flops": fl.value, "bytes": by.value}


class VGroup:
    """In-process virtual ranks on one device (rg_vgroup_create): P handles, one host thread per
    rank, run the library's row-sharded code path with fixed-order on-device collectives."""

    def __init__(self, nranks: int, device: int = 0):
        import torch
        torch.cuda.set_device(device)
        self._g = ctypes.c_void_p()
        st = _lib().rg_vgroup_create(ctypes.byref(self._g), int(nranks))
        if st != RG_OK:
            raise RGError("rg_vgroup_create", st)
        self.nranks = nranks
        self.device = device

    @property
    def ptr(self):
        return self._g

    def close(self):
        if self._g:
            _lib().rg_vgroup_destroy(self._g)
            self._g = ctypes.c_void_p()


def run_ranks(fns):
    """Run fns[r]() on one host thread per rank (the library releases the GIL in every call);
    returns their results, re-raising the first exception."""
    import threading
    out = [None] * len(fns)
    err = [None] * len(fns)

    def body(r):
        try:
            out[r] = fns[r]()
        except BaseException as e:  # noqa: BLE001
            err[r] = e

    ts = [threading.Thread(target=body, args=(r,)) for r in range(len(fns))]
    for t in ts:
        t.start()
    for t in ts:
        t.join()
    for e in err:
        if e is not None:
            raise e
    return out


def debug_gaussian(n: int, seed: int, out=None, handle=None):
    """The device Philox4x32-10 + Box-Muller generator behind lowrank_approx's Omega and the
    Hutchinson probes, exposed for bit-exact parity tests: n fp64 values into a CUDA tensor."""
    import torch
    h = _handle(handle)
    if out is None:
        out = torch.empty(n, dtype=torch.float64, device="cuda")
    _check("rg_debug_gaussian", _lib().rg_debug_gaussian(h.ptr, int(n), ctypes.c_uint64(int(seed) & (2**64 - 1)),
                                                        ctypes.c_void_p(out.data_ptr())), h)
    return out


def debug_philox(ncalls: int, seed: int, handle=None):
    """Raw Philox4x32-10 words (ncalls x 4 uint32 as int64 numpy) of the device generator."""
    import torch
    h = _handle(handle)
    out = torch.empty(ncalls * 4, dtype=torch.int32, device="cuda")
    _check("rg_debug_philox", _lib().rg_debug_philox(h.ptr, int(ncalls), ctypes.c_uint64(int(seed) & (2**64 - 1)),
                                                    ctypes.c_void_p(out.data_ptr())), h)
    return out.cpu().numpy().view(np.uint32).astype(np.int64).reshape(ncalls, 4)


def _find_nccl():
    try:
        import nvidia.nccl
        for base in nvidia.nccl.__path__:
            p = os.path.join(base, "lib", "libnccl.so.2")
            if os.path.exists(p):
                return p
    except Exception:
        pass
    return None


def _check(func, st, h=None):
    if st != RG_OK:
        info = h.last_info() if isinstance(h, Handle) else -1
        raise RGError(func, st, info)


_default_handles: dict = {}


def default_handle(device=None) -> Handle:
    import torch
    if device is None:
        device = torch.cuda.current_device()
    h = _default_handles.get(device)
    if h is None:
        h = Handle(device)
        _default_handles[device] = h
    return h


def _handle(h):
    return h if h is not None else default_handle()


# ======================================================================= API
def rgsqr_factor(A, Q=None, R=None, *, handle=None, opts: rg_opts | None = None, check=True):
    """A = Q R (Algorithm 1).  A: m x n column-major fp32 (torch CUDA tensor or numpy F array).
    Q defaults to a new column-major buffer (pass Q=A to factor in place); R: n x n.
    Returns (Q, R).  Raises RGError on breakdown / non-finite input."""
    h = _handle(handle)
    a = _mat(A, "A")
    m, n = a.rows, a.cols
    if Q is None:
        Q = _like(A, m, n)
    if R is None:
        R = _like(A, n, n)
    q, r = _mat(Q, "Q"), _mat(R, "R")
    o = opts if opts is not None else make_opts()
    st = _lib().rgsqr_factor(h.ptr, m, n, ctypes.c_void_p(a.ptr), a.ld, ctypes.c_void_p(q.ptr), q.ld,
                             ctypes.c_void_p(r.ptr), r.ld, ctypes.byref(o))
    if check:
        _check("rgsqr_factor", st, h)
    return Q, R


def orthogonalize(A, R=None, *, orth_tol=1e-5, max_passes=2, handle=None, opts=None, check=True):
    """Overwrite A (m x n) by Q with orthonormal columns (section 3.3).  Returns
    (A, R, passes, orth_est)."""
    h = _handle(handle)
    a = _mat(A, "A")
    r = _mat(R, "R") if R is not None else None
    passes = ctypes.c_int(0)
    est = ctypes.c_double(0.0)
    o = opts if opts is not None else make_opts()
    st = _lib().orthogonalize(h.ptr, a.rows, a.cols, ctypes.c_void_p(a.ptr), a.ld,
                              ctypes.c_void_p(r.ptr if r else 0), r.ld if r else a.cols, float(orth_tol),
                              int(max_passes), ctypes.byref(passes), ctypes.byref(est), ctypes.byref(o))
    if check and st not in (RG_OK,):
        _check("orthogonalize", st, h)
    return A, R, passes.value, est.value


def ls_solve_refined(A, b, x=None, *, tol=1e-10, maxit=200, handle=None, opts=None, check=True):
    """x = argmin ||A x - b|| via RGSQR + R-preconditioned CGLS (Alg 3 corrected).
    Returns (x fp64, iters, relres, status)."""
    h = _handle(handle)
    a = _mat(A, "A")
    bb = _mat(b, "b")
    if x is None:
        x = _like(A, a.cols, None, dtype="float64")
    xx = _mat(x, "x", dtype="float64")
    it = ctypes.c_int(0)
    rel = ctypes.c_double(0.0)
    o = opts if opts is not None else make_opts()
    st = _lib().ls_solve_refined(h.ptr, a.rows, a.cols, ctypes.c_void_p(a.ptr), a.ld, ctypes.c_void_p(bb.ptr),
                                 ctypes.c_void_p(xx.ptr), float(tol), int(maxit), ctypes.byref(it),
                                 ctypes.byref(rel), ctypes.byref(o))
    if check and st not in (RG_OK, RG_NOT_CONVERGED):
        _check("ls_solve_refined", st, h)
    return x, it.value, rel.value, st


def lowrank_approx(A, rank, *, oversample=16, power_iters=1, seed=0, U=None, S=None, V=None, handle=None,
                   opts=None, check=True):
    """Randomized rank-`rank` approximation A ~ U diag(S) V^T (RGSQR range finder)."""
    h = _handle(handle)
    a = _mat(A, "A")
    m, n = a.rows, a.cols
    if U is None:
        U = _like(A, m, rank)
    if S is None:
        S = _like(A, rank, None)
    if V is None:
        V = _like(A, n, rank)
    u, s, v = _mat(U, "U"), _mat(S, "S"), _mat(V, "V")
    o = opts if opts is not None else make_opts()
    st = _lib().lowrank_approx(h.ptr, m, n, ctypes.c_void_p(a.ptr), a.ld, int(rank), int(oversample),
                               int(power_iters), ctypes.c_uint64(int(seed) & 0xFFFFFFFFFFFFFFFF),
                               ctypes.c_void_p(u.ptr), u.ld, ctypes.c_void_p(s.ptr), ctypes.c_void_p(v.ptr), v.ld,
                               ctypes.byref(o))
    if check:
        _check("lowrank_approx", st, h)
    return U, S, V


def lowrank_qrsvd(A, rank, *, U=None, S=None, V=None, handle=None, opts=None, check=True):
    """Deterministic QR-SVD rank-`rank` approximation of a tall-skinny A (section 3.4, Table 4):
    A = QR, R = U_R S V_R^T, U = Q U_R(:, :rank).  Returns (U, S, V)."""
    h = _handle(handle)
    a = _mat(A, "A")
    m, n = a.rows, a.cols
    if U is None:
        U = _like(A, m, rank)
    if S is None:
        S = _like(A, rank, None)
    if V is None:
        V = _like(A, n, rank)
    u, s, v = _mat(U, "U"), _mat(S, "S"), _mat(V, "V")
    o = opts if opts is not None else make_opts()
    st = _lib().lowrank_qrsvd(h.ptr, m, n, ctypes.c_void_p(a.ptr), a.ld, int(rank), ctypes.c_void_p(u.ptr), u.ld,
                              ctypes.c_void_p(s.ptr), ctypes.c_void_p(v.ptr), v.ld, ctypes.byref(o))
    if check:
        _check("lowrank_qrsvd", st, h)
    return U, S, V


def _like(ref, rows, cols, dtype="float32"):
    if isinstance(ref, np.ndarray):
        shape = (rows,) if cols is None else (rows, cols)
        return np.zeros(shape, dtype=dtype, order="F")
    import torch
    dt = {"float32": torch.float32, "float64": torch.float64}[dtype]
    if cols is None:
        return torch.zeros(rows, dtype=dt, device=ref.device)
    return torch.zeros(cols, rows, dtype=dt, device=ref.device).t()
