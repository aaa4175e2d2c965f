"""NEXT-1: deterministic QR-SVD low rank of a tall-skinny matrix, section 3.4
(P:L328-355), through the C-ABI lowrank_qrsvd (-m gpu).

* Table 4 at the paper's size (524288 x 1024, arithmetic singular values, cond 1e6): the
  relative Frobenius error ||A - U S V^T|| / ||A|| equals the printed value (tests/golden/
  table4_lowrank.txt, 3 significant digits) for r = 16 .. 512, and S the constructed spectrum.
* Parity at a small size against the oracle's own QR-SVD (fp64 Householder + one-sided Jacobi):
  same truncation errors, same singular values, orthonormal factors.
"""
import os

import numpy as np
import pytest

import oracle
import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

GOLD = os.path.join(os.path.dirname(__file__), "golden", "table4_lowrank.txt")


@pytest.fixture(scope="module")
def rg():
    import paper_conf_hpdc_zhangbw20_b200 as rg
    return rg


def _golden():
    rows = []
    for line in open(GOLD):
        line = line.strip()
        if line and not line.startswith("#"):
            r, a, b = line.split()
            rows.append((int(r), float(a), float(b)))
    return rows


def _dev(A):
    return torch.from_numpy(np.ascontiguousarray(np.asarray(A, dtype=np.float32).T)).cuda().t()


def test_qrsvd_table4_full_size(rg):
    m, n = 524288, 1024
    At, s = synth.svd_matrix_device(m, n, "arithmetic", 1e6, seed=4)
    A = At.t()
    nrmA = torch.linalg.norm(At.double()).item()
    h = rg.Handle(0)
    for r, printed, _ in _golden():
        U, S, V = rg.lowrank_qrsvd(A, r, handle=h)
        torch.cuda.synchronize()
        # ||A - U S V^T||_F in fp64 on the device, in row blocks (check only)
        num = 0.0
        Us = U.double() * S.double()
        Vt = V.double().t()
        for i0 in range(0, m, 65536):
            num += torch.linalg.norm(A[i0:i0 + 65536].double() - Us[i0:i0 + 65536] @ Vt).item() ** 2
        err = np.sqrt(num) / nrmA
        assert f"{err:.2e}" == f"{printed:.2e}", (r, err, printed)
        np.testing.assert_allclose(S.cpu().numpy(), s[:r], rtol=1e-4)
        assert np.all(np.diff(S.cpu().numpy()) <= 0)
        Vn = V.cpu().numpy().astype(np.float64)
        assert np.linalg.norm(Vn.T @ Vn - np.eye(r)) < 1e-4
        G = (U.double().t() @ U.double()).cpu().numpy()
        assert np.linalg.norm(G - np.eye(r)) < 1e-2 * np.sqrt(r)   # first-pass Q (no reortho)
    h.close()


@pytest.mark.parametrize("kind,kappa", [("arithmetic", 1e6), ("geometric", 1e3)])
def test_qrsvd_matches_oracle(rg, kind, kappa):
    m, n, r = 6000, 256, 48
    A = synth.svd_matrix(m, n, kind, kappa, seed=71).astype(np.float32)
    A64 = A.astype(np.float64)
    U, S, V = rg.lowrank_qrsvd(_dev(A), r)
    U, S, V = (x.cpu().numpy().astype(np.float64) for x in (U, S, V))
    # oracle QR-SVD in fp64: Householder R, Jacobi SVD of R (the same algorithm, no 16-bit rounding)
    Qo, Ro, _ = oracle.householder(A64)
    Ur, So, Vr, _ = oracle.svd_jacobi(Ro)
    order = np.argsort(-So)
    Ur, So, Vr = Ur[:, order], So[order], Vr[:, order]
    Uo = Qo @ Ur[:, :r]
    err = oracle.lowrank_error(A64, U, S, V)
    err_o = oracle.lowrank_error(A64, Uo, So[:r], Vr[:, :r])
    s = synth.sigma(n, kind, kappa)
    opt = np.sqrt(np.sum(s[r:] ** 2) / np.sum(s ** 2))
    assert abs(err_o - opt) <= 1e-10
    assert abs(err - err_o) <= 1e-4 * err_o, (err, err_o)
    np.testing.assert_allclose(S, So[:r], rtol=2e-4)
    assert np.linalg.norm(V.T @ V - np.eye(r)) < 1e-4


def test_qrsvd_argument_checks(rg):
    import ctypes
    h = rg.default_handle()
    L = rg.lib()
    o = rg.make_opts()
    A = torch.zeros(100, 20, device="cuda")
    p = ctypes.c_void_p(A.data_ptr())
    assert L.lowrank_qrsvd(h.ptr, 100, 20, p, 100, 0, p, 100, p, p, 20, ctypes.byref(o)) == -6
    assert L.lowrank_qrsvd(h.ptr, 100, 20, p, 100, 21, p, 100, p, p, 20, ctypes.byref(o)) == -6
    assert L.lowrank_qrsvd(h.ptr, 100, 20, p, 100, 5, p, 99, p, p, 20, ctypes.byref(o)) == -8
    assert L.lowrank_qrsvd(h.ptr, 100, 20, p, 100, 5, p, 100, p, p, 19, ctypes.byref(o)) == -11
