"""GPU parity at BASELINE.json's full sizes, in the launch configuration bench.py times (-m gpu).

The oracle cannot factor 65536 x 4096 in seconds, so at full size the checks are
  * sampled outputs the oracle computes directly: the thin QR of a full-rank matrix is unique
    (positive diag R) and the QR of the leading k columns A[:, :k] is exactly
    (Q[:, :k], R[:k, :k]) -- the oracle's Householder QR of A[:, :k] pins those entries;
  * properties that hold at any size, evaluated exactly (fp64 products on the device, check
    only, not the product path): ||A - QR||_F / ||A||_F, ||I - Q^T Q||_F, triangularity,
    positive diagonal; for least squares the fp64 normal-equations solution of the oracle;
    for low rank the closed-form optimal truncation error of the constructed spectrum.
Tolerances are the north_star's.
"""
import numpy as np
import pytest

import oracle
import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def rg():
    import paper_conf_hpdc_zhangbw20_b200 as rg
    return rg


def _exact_metrics(A, Q, R):
    """fp64 ||A - QR||_F/||A||_F and ||I - Q^T Q||_F of device tensors (chunked over columns)."""
    n = Q.shape[1]
    Q64 = Q.double()
    G = Q64.t() @ Q64
    orth = torch.linalg.norm(G - torch.eye(n, dtype=torch.float64, device=G.device)).item()
    del G
    R64 = R.double()
    num = 0.0
    den = 0.0
    for j0 in range(0, n, 512):
        j1 = min(n, j0 + 512)
        Aj = A[:, j0:j1].double()
        num += torch.linalg.norm(Aj - Q64 @ R64[:, j0:j1]).item() ** 2
        den += torch.linalg.norm(Aj).item() ** 2
    return (num / den) ** 0.5, orth


def _leading_block_check(A_host, Q, R, k, tol):
    """(Q[:, :k], R[:k, :k]) against the oracle's Householder QR of A[:, :k] (unique)."""
    Ak = np.asarray(A_host[:, :k], dtype=np.float64)
    Qo, Ro, _ = oracle.householder(Ak)
    Rg = R[:k, :k].double().cpu().numpy()
    Qg = Q[:, :k].double().cpu().numpy()
    dr = np.linalg.norm(Rg - Ro) / np.linalg.norm(Ro)
    dq = np.linalg.norm(Qg - Qo) / np.linalg.norm(Qo)
    assert dr <= tol and dq <= tol, (k, dr, dq)
    return dr, dq


def test_config2_full_size(rg):
    """C2: RGSQR of 65536 x 4096 fp32 N(0,1), fp16 tensor-core updates, bench.py's options
    (make_opts(sync=False), leaf/plan chosen by the library exactly as in the timed call)."""
    m, n = 65536, 4096
    A_host = synth.gaussian(m, n, seed=synth.SEED_BASE + 1, dtype=np.float32)
    A = torch.from_numpy(np.ascontiguousarray(A_host.T)).cuda().t()
    h = rg.Handle(0)
    opts = rg.make_opts(sync=False)
    Q = torch.empty(n, m, device="cuda").t()
    R = torch.empty(n, n, device="cuda").t()
    for _ in range(2):   # second call replays the captured plan, like bench.py's timed steps
        rg.rgsqr_factor(A, Q=Q, R=R, handle=h, opts=opts, check=False)
    torch.cuda.synchronize()
    assert torch.isfinite(Q).all() and torch.isfinite(R).all()
    assert (torch.tril(R, -1) == 0).all()
    assert (torch.diagonal(R) > 0).all()
    be, orth = _exact_metrics(A, Q, R)
    assert be <= 5e-3, be
    assert orth <= 1e-2 * np.sqrt(n), orth
    # expected be ~5e-5, orth_F ~6e-3 at this shape
    # leading 64 (one leaf) and 192 (leaf + folded level + one tcgen05 K1/K2 level) columns
    for k in (64, 192):
        _leading_block_check(A_host, Q, R, k, tol=10 * 1.7 * (be + orth / np.sqrt(n)) + 1e-5)
    # a sampled trailing column: R[:, j] = Q^T a_j for the unique factors, so with the GPU's own
    # (near-orthonormal) Q the last column of R matches Q^T a_j to the backward error
    j = n - 1
    r_j = (Q.double().t() @ A[:, j].double())
    d = torch.linalg.norm(r_j - R[:, j].double()) / torch.linalg.norm(R[:, j].double())
    assert d.item() <= 10 * (be + orth), d.item()
    h.close()


def test_config3_full_size(rg):
    """C3: least squares 131072 x 1024, cond 1e4 geometric, R-preconditioned CGLS, both right-hand
    sides (reading #16); x* from the oracle's fp64 normal equations (kappa^2 u64 ~ 1e-8)."""
    m, n = 131072, 1024
    A = synth.svd_matrix(m, n, "geometric", 1e4, seed=synth.SEED_BASE + 2).astype(np.float32)
    A64 = A.astype(np.float64)
    Ad = torch.from_numpy(np.ascontiguousarray(A.T)).cuda().t()
    for consistent in (False, True):
        b = synth.rhs(A64, seed=synth.SEED_BASE + 2, consistent=consistent).astype(np.float32)
        x_star, st0 = oracle.ls_normal(A64, b.astype(np.float64))
        assert st0 == 0
        x = torch.zeros(n, dtype=torch.float64, device="cuda")
        x, it, rel, st = rg.ls_solve_refined(Ad, torch.from_numpy(b).cuda(), x, tol=1e-10, maxit=200)
        fe = np.linalg.norm(x.cpu().numpy() - x_star) / np.linalg.norm(x_star)
        assert st == rg.RG_OK, (st, it, rel)
        assert fe <= 1e-5, (consistent, fe, it)
        assert it <= 60, it


def test_config4_full_size(rg):
    """C4: orthogonalisation of 2,097,152 x 256 N(0,1) with reorthogonalisation; exact fp64
    orthogonality <= 1e-5 and backward error <= 5e-3."""
    m, n = 2097152, 256
    g = torch.Generator(device="cuda").manual_seed(synth.SEED_BASE + 4)
    A = torch.randn(n, m, generator=g, device="cuda", dtype=torch.float32).t()
    A0 = A.clone()
    R = torch.zeros(n, n, device="cuda").t()
    Q, R, passes, est = rg.orthogonalize(A, R, orth_tol=1e-5, max_passes=3)
    torch.cuda.synchronize()
    be, orth = _exact_metrics(A0, Q, R)
    assert orth <= 1e-5, (orth, passes, est)
    assert be <= 5e-3, be
    assert 1 <= passes <= 3
    # sampled outputs: the unique QR of the leading 64 columns (one leaf) from the oracle
    A_lead = A0[:, :64].cpu().numpy()
    _leading_block_check(A_lead, Q, R, 64, tol=1e-4)


def test_config5_full_size(rg):
    """C5: randomized low rank of 32768 x 32768 at rank 512 (p = 16, q = 1) via the RGSQR range
    finder; A = U_k diag(sigma) V_k^T (k = 2048, geometric 1 -> 1e-6) so the optimal rank-512
    Frobenius error is closed-form; reading #17: ratio ~1.016 with q = 1."""
    m = n = 32768
    k, rank = 2048, 512
    At, s = synth.lowrank_matrix(m, n, k, "geometric", 1e6, seed=synth.SEED_BASE + 5, device="cuda")
    A = At.t()                      # column-major m x n view
    U, S, V = rg.lowrank_approx(A, rank, oversample=16, power_iters=1, seed=7)
    torch.cuda.synchronize()
    Sn = S.double().cpu().numpy()
    assert np.all(np.diff(Sn) <= 0) and np.all(Sn > 0)
    np.testing.assert_allclose(Sn[:64], s[:64], rtol=2e-3)
    # ||A - U S V^T||_F in fp64, chunked over columns
    U64, V64, S64 = U.double(), V.double(), S.double()
    num = 0.0
    for j0 in range(0, n, 4096):
        Aj = A[:, j0:j0 + 4096].double()
        num += torch.linalg.norm(Aj - (U64 * S64) @ V64[j0:j0 + 4096].t()).item() ** 2
    err = (num / np.sum(s ** 2)) ** 0.5
    opt = np.sqrt(np.sum(s[rank:] ** 2) / np.sum(s ** 2))
    assert err >= opt * (1 - 1e-6)
    # the spectrum decays slowly across the oversampling window (sigma_528 / sigma_512 = 0.989),
    # so one power iteration leaves ~5 % above the optimum here (measured 1.054 with seed 7;
    # the scaled case in test_gpu_lowrank reaches ~1.016); bound at 1.10
    assert err / opt < 1.10, (err, opt)
