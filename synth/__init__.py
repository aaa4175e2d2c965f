"""Seeded synthetic input generators shared by the oracle side and the CUDA side.

This module holds NO arithmetic of the method (no QR of the input, no
Gram-Schmidt, no least squares); it only draws test matrices with the
spectra of the paper's workloads (section 4.2; reading #15 in
DESIGN.md) so both sides see identical inputs:

* ``gaussian``      -- i.i.d. N(0,1)                       (P:L405 type 2)
* ``uniform``       -- i.i.d. U(0,1) or U(-1,1)             (P:L405 type 1)
* ``svd_matrix``    -- A = U diag(sigma) V^T with Haar U (m x n), V (n x n) and
  sigma "geometric" (log sigma evenly spaced, type 3), "arithmetic" (sigma evenly
  spaced, type 4) or "cluster" (all 1 but the smallest = 1/kappa, type 5),
  sigma_1 = 1, sigma_n = 1/kappa.
* ``lowrank_matrix`` -- A = U_k diag(sigma) V_k^T with k < min(m, n) (config 5).
* ``rhs``           -- b ~ N(0,1) (inconsistent) or b = A x_true (reading #16).

Seeds: ``SEED_BASE + config_index`` with numpy PCG64.
Haar factors are drawn as the sign-fixed orthonormal factor of a Gaussian
matrix (numpy/LAPACK; a generator detail, not the method under test).
"""
from __future__ import annotations

import numpy as np

SEED_BASE = 20200623


def rng(seed: int) -> np.random.Generator:
    return np.random.Generator(np.random.PCG64(int(seed)))


def gaussian(m: int, n: int, seed: int, dtype=np.float64) -> np.ndarray:
    g = rng(seed)
    return np.asfortranarray(g.standard_normal((n, m), dtype=np.float64).T.astype(dtype, copy=False))


def uniform(m: int, n: int, seed: int, low: float = 0.0, high: float = 1.0, dtype=np.float64) -> np.ndarray:
    g = rng(seed)
    return np.asfortranarray(g.uniform(low, high, size=(n, m)).T.astype(dtype, copy=False))


def sigma(n: int, kind: str, kappa: float) -> np.ndarray:
    """Singular values sigma_1 = 1 >= ... >= sigma_n = 1/kappa."""
    i = np.arange(n, dtype=np.float64)
    if n == 1:
        return np.ones(1)
    if kind == "geometric":
        return kappa ** (-i / (n - 1))
    if kind == "arithmetic":
        return 1.0 - i / (n - 1) * (1.0 - 1.0 / kappa)
    if kind == "cluster":
        s = np.ones(n)
        s[-1] = 1.0 / kappa
        return s
    raise ValueError(f"unknown spectrum kind {kind!r}")


def haar(m: int, n: int, g: np.random.Generator) -> np.ndarray:
    """m x n with orthonormal columns, Haar distributed (sign-fixed Gaussian QR)."""
    X = g.standard_normal((m, n))
    Q, R = np.linalg.qr(X)
    d = np.sign(np.diag(R))
    d[d == 0] = 1.0
    return np.asfortranarray(Q * d)


def svd_matrix(m: int, n: int, kind: str, kappa: float, seed: int, dtype=np.float64) -> np.ndarray:
    g = rng(seed)
    U = haar(m, n, g)
    V = haar(n, n, g)
    s = sigma(n, kind, kappa)
    return np.asfortranarray(((U * s) @ V.T).astype(dtype, copy=False))


def lowrank_matrix(m: int, n: int, k: int, kind: str, kappa: float, seed: int, device=None):
    """A = U_k diag(sigma) V_k^T (rank k).  Returns (A fp32, sigma).  With a torch
    `device` the outer product runs there in fp64 (test-harness cost only)."""
    g = rng(seed)
    U = haar(m, k, g)
    V = haar(n, k, g)
    s = sigma(k, kind, kappa)
    if device is None:
        A = np.asfortranarray(((U * s) @ V.T).astype(np.float32))
        return A, s
    import torch

    Ut = torch.from_numpy(U * s).to(device)
    Vt = torch.from_numpy(np.ascontiguousarray(V)).to(device)
    # column-major A (m x n) == row-major A^T (n x m) = V (U s)^T
    At = (Vt @ Ut.T).to(torch.float32).contiguous()
    return At, s


def svd_matrix_device(m: int, n: int, kind: str, kappa: float, seed: int, device="cuda"):
    """Large-size form of svd_matrix for the GPU tests / bench (test-harness cost only): the
    Gaussian factors are drawn with a seeded torch generator ON the device and orthonormalised
    there (fp64); same spectrum recipe (reading #15).  Returns (A^T row-major fp32 (n x m), i.e.
    column-major A, and sigma)."""
    import torch

    gen = torch.Generator(device=device).manual_seed(int(seed))
    X = torch.randn(m, n, generator=gen, device=device, dtype=torch.float64)
    U, Ru = torch.linalg.qr(X)
    U *= torch.sign(torch.diagonal(Ru))
    del X, Ru
    Y = torch.randn(n, n, generator=gen, device=device, dtype=torch.float64)
    V, Rv = torch.linalg.qr(Y)
    V *= torch.sign(torch.diagonal(Rv))
    s = sigma(n, kind, kappa)
    U *= torch.from_numpy(s).to(device)
    At = (V @ U.T).to(torch.float32).contiguous()   # (U s V^T)^T
    del U, V, Y
    return At, s


def rhs(A: np.ndarray, seed: int, consistent: bool) -> np.ndarray:
    g = rng(seed + 7919)
    m, n = A.shape
    if consistent:
        x = g.standard_normal(n)
        return np.asarray(A, dtype=np.float64) @ x
    return g.standard_normal(m)


def probes(n: int, p: int, seed: int) -> np.ndarray:
    """Hutchinson probe vectors G (n x p), N(0,1)."""
    return gaussian(n, p, seed + 104729)
