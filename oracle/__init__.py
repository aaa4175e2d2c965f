"""fp64 CPU oracle for the RGSQR hot path (ctypes binding of oracle/oracle.c).

TEST INFRASTRUCTURE ONLY.  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import this
package.  The product package ``paper_conf_hpdc_zhangbw20_b200`` never imports
it, and the two share no code ("Oracle").

Every function takes/returns numpy float64 arrays in Fortran (column-major)
order and follows a passage of PAPER.md ("P:Lnnn"):

* ``cgs``/``mgs``/``householder`` -- the unique thin QR with positive diag(R)
  (P:L91); ``mgs`` is Algorithm 2 verbatim.
* ``tsqr`` -- the CAQR panel of eq 8 with MGS tiles.
* ``rgsqr`` -- Algorithm 1 with the TSQR leaf, reading #1.
* ``ls_normal`` (eq 2), ``ls_qr`` (eq 3), ``cgls`` (Alg 3,
  P:L280-301, corrected per readings #5/#6).
* metrics of P:L262/L268/L336 (Frobenius, reading #12) and Hutchinson probes.
* ``svd_jacobi``, ``lowrank`` (QR-SVD of section 3.4; randomized range
  finder of BASELINE config 5, reading #17), ``gaussian_philox`` (the
  counter-based sketch generator, restated independently on the device).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

_f64p = np.ctypeslib.ndpointer(dtype=np.float64, flags="F_CONTIGUOUS")
_f64v = np.ctypeslib.ndpointer(dtype=np.float64, flags="C_CONTIGUOUS")
_i64 = ctypes.c_int64


def build(force: bool = False) -> str:
    """Compile liboracle.so with plain gcc (-O2, IEEE fp64, OpenMP)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(
            ["gcc", "-O2", "-std=c11", "-fopenmp", "-fPIC", "-shared", "-fno-fast-math",
             "-ffp-contract=off", _SRC, "-o", _LIB, "-lm"])
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build())
        L = _lib
        qr_sig = [_i64, _i64, _f64p, _i64, _f64p, _i64, _f64p, _i64]
        for name in ("or_cgs", "or_mgs", "or_householder"):
            getattr(L, name).argtypes = qr_sig
            getattr(L, name).restype = ctypes.c_int
        L.or_tsqr.argtypes = qr_sig + [_i64]
        L.or_tsqr.restype = ctypes.c_int
        L.or_rgsqr.argtypes = qr_sig + [_i64, _i64]
        L.or_rgsqr.restype = ctypes.c_int
        L.or_rgsqr_split.argtypes = [_i64]
        L.or_rgsqr_split.restype = _i64
        L.or_rgsqr_flops.argtypes = [_i64, _i64, _i64]
        L.or_rgsqr_flops.restype = ctypes.c_double
        L.or_matmul.argtypes = [_i64, _i64, _i64, _f64p, _i64, _f64p, _i64, _f64p, _i64]
        L.or_matmul_tn.argtypes = [_i64, _i64, _i64, _f64p, _i64, _f64p, _i64, _f64p, _i64]
        L.or_trsv_upper.argtypes = [_i64, _f64p, _i64, _f64v]
        L.or_trsv_upper_t.argtypes = [_i64, _f64p, _i64, _f64v]
        L.or_ls_normal.argtypes = [_i64, _i64, _f64p, _i64, _f64v, _f64v]
        L.or_ls_normal.restype = ctypes.c_int
        L.or_ls_qr.argtypes = [_i64, _i64, _f64p, _i64, _f64v, _f64v]
        L.or_ls_qr.restype = ctypes.c_int
        L.or_cgls.argtypes = [_i64, _i64, _f64p, _i64, _f64v, _f64p, _i64, ctypes.c_double,
                              ctypes.c_int, _f64v, ctypes.POINTER(ctypes.c_double)]
        L.or_cgls.restype = ctypes.c_int
        L.or_backward_error.argtypes = [_i64, _i64, _f64p, _i64, _f64p, _i64, _f64p, _i64]
        L.or_backward_error.restype = ctypes.c_double
        L.or_orthogonality.argtypes = [_i64, _i64, _f64p, _i64]
        L.or_orthogonality.restype = ctypes.c_double
        L.or_lowrank_error.argtypes = [_i64, _i64, _i64, _f64p, _i64, _f64p, _i64, _f64v, _f64p, _i64]
        L.or_lowrank_error.restype = ctypes.c_double
        L.or_backward_error_probe.argtypes = [_i64, _i64, _f64p, _i64, _f64p, _i64, _f64p, _i64,
                                              ctypes.c_int, _f64p]
        L.or_backward_error_probe.restype = ctypes.c_double
        L.or_orthogonality_probe.argtypes = [_i64, _i64, _f64p, _i64, ctypes.c_int, _f64p]
        L.or_orthogonality_probe.restype = ctypes.c_double
        L.or_svd_jacobi.argtypes = [_i64, _i64, _f64p, _i64, _f64p, _i64, _f64v, _f64p, _i64]
        L.or_svd_jacobi.restype = ctypes.c_int
        L.or_lowrank.argtypes = [_i64, _i64, _f64p, _i64, _i64, _i64, ctypes.c_int, _f64p,
                                 _f64p, _i64, _f64v, _f64p, _i64]
        L.or_lowrank.restype = ctypes.c_int
        L.or_philox4x32_10.argtypes = [ctypes.POINTER(ctypes.c_uint32), ctypes.POINTER(ctypes.c_uint32),
                                       ctypes.POINTER(ctypes.c_uint32)]
        L.or_gaussian_philox.argtypes = [_i64, _i64, ctypes.c_uint64, _f64p]
    return _lib


def _f(a) -> np.ndarray:
    return np.asfortranarray(np.asarray(a, dtype=np.float64))


def _qr(fn, A, *extra):
    A = _f(A)
    m, n = A.shape
    Q = np.zeros((m, n), order="F")
    R = np.zeros((n, n), order="F")
    status = getattr(lib(), fn)(m, n, A, m, Q, m, R, n, *extra)
    return Q, R, status


def cgs(A):
    """Classical Gram-Schmidt. Returns (Q, R, status)."""
    return _qr("or_cgs", A)


def mgs(A):
    """Modified Gram-Schmidt, Algorithm 2. Returns (Q, R, status)."""
    return _qr("or_mgs", A)


def householder(A):
    """Sign-normalised Householder QR. Returns (Q, R, status)."""
    return _qr("or_householder", A)


def tsqr(A, tile=256):
    """CAQR/TSQR panel, eq 8 with MGS tiles of `tile` rows."""
    return _qr("or_tsqr", A, int(tile))


def rgsqr(A, nb=32, tile=256):
    """Algorithm 1 in fp64, leaf = TSQR when n <= nb."""
    return _qr("or_rgsqr", A, int(nb), int(tile))


def rgsqr_split(n: int) -> int:
    return int(lib().or_rgsqr_split(int(n)))


def rgsqr_flops(m: int, n: int, nb: int) -> float:
    """Recurrence eq 5."""
    return float(lib().or_rgsqr_flops(int(m), int(n), int(nb)))


def matmul(A, B):
    A, B = _f(A), _f(B)
    m, n = A.shape
    k = B.shape[1]
    C = np.zeros((m, k), order="F")
    lib().or_matmul(m, n, k, A, m, B, n, C, m)
    return C


def trsv_upper(R, x, transpose=False):
    R = _f(R)
    x = np.ascontiguousarray(np.array(x, dtype=np.float64))
    n = R.shape[0]
    (lib().or_trsv_upper_t if transpose else lib().or_trsv_upper)(n, R, n, x)
    return x


def ls_normal(A, b):
    A = _f(A)
    m, n = A.shape
    x = np.zeros(n)
    s = lib().or_ls_normal(m, n, A, m, np.ascontiguousarray(b, dtype=np.float64), x)
    return x, s


def ls_qr(A, b):
    A = _f(A)
    m, n = A.shape
    x = np.zeros(n)
    s = lib().or_ls_qr(m, n, A, m, np.ascontiguousarray(b, dtype=np.float64), x)
    return x, s


def cgls(A, b, R, tol=1e-10, maxit=200):
    """Algorithm 3 corrected (readings #5/#6). Returns (x, iters, relres)."""
    A, R = _f(A), _f(R)
    m, n = A.shape
    x = np.zeros(n)
    rel = ctypes.c_double(0.0)
    it = lib().or_cgls(m, n, A, m, np.ascontiguousarray(b, dtype=np.float64), R, n,
                       float(tol), int(maxit), x, ctypes.byref(rel))
    return x, int(it), rel.value


def backward_error(A, Q, R):
    A, Q, R = _f(A), _f(Q), _f(R)
    m, n = A.shape
    return float(lib().or_backward_error(m, n, A, m, Q, m, R, n))


def orthogonality(Q):
    Q = _f(Q)
    m, n = Q.shape
    return float(lib().or_orthogonality(m, n, Q, m))


def lowrank_error(A, U, S, V):
    A, U, V = _f(A), _f(U), _f(V)
    m, n = A.shape
    r = U.shape[1]
    return float(lib().or_lowrank_error(m, n, r, A, m, U, m, np.ascontiguousarray(S, dtype=np.float64), V, n))


def backward_error_probe(A, Q, R, G):
    """Hutchinson estimate of ||A-QR||_F/||A||_F with probe matrix G (n x p)."""
    A, Q, R, G = _f(A), _f(Q), _f(R), _f(G)
    m, n = A.shape
    return float(lib().or_backward_error_probe(m, n, A, m, Q, m, R, n, G.shape[1], G))


def orthogonality_probe(Q, G):
    Q, G = _f(Q), _f(G)
    m, n = Q.shape
    return float(lib().or_orthogonality_probe(m, n, Q, m, G.shape[1], G))


def svd_jacobi(A):
    A = _f(A)
    m, n = A.shape
    U = np.zeros((m, n), order="F")
    V = np.zeros((n, n), order="F")
    S = np.zeros(n)
    sweeps = lib().or_svd_jacobi(m, n, A, m, U, m, S, V, n)
    return U, S, V, sweeps


def lowrank(A, rank, oversample, power_iters, Omega):
    A, Omega = _f(A), _f(Omega)
    m, n = A.shape
    l = rank + oversample
    assert Omega.shape == (n, l)
    U = np.zeros((m, rank), order="F")
    V = np.zeros((n, rank), order="F")
    S = np.zeros(rank)
    s = lib().or_lowrank(m, n, A, m, rank, l, int(power_iters), Omega, U, m, S, V, n)
    return U, S, V, s


def philox4x32_10(ctr, key):
    c = (ctypes.c_uint32 * 4)(*[int(v) & 0xFFFFFFFF for v in ctr])
    k = (ctypes.c_uint32 * 2)(*[int(v) & 0xFFFFFFFF for v in key])
    o = (ctypes.c_uint32 * 4)()
    lib().or_philox4x32_10(c, k, o)
    return [int(v) for v in o]


def gaussian_philox(rows, cols, seed):
    out = np.zeros((rows, cols), order="F")
    lib().or_gaussian_philox(int(rows), int(cols), int(seed) & 0xFFFFFFFFFFFFFFFF, out)
    return out
